#!/usr/bin/env python
"""Key metrics of every kernel in an ncu report (--set full) as JSON.

    python tools/ncu_summary.py gpurun_out/prof.ncu-rep > profiles/r01_<name>.json
"""
import csv
import io
import json
import subprocess
import sys

WANT = {
    "gpu__time_duration.sum": "duration_ns",
    "dram__bytes_read.sum": "dram_read_bytes",
    "dram__bytes_write.sum": "dram_write_bytes",
    "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed": "dram_pct_of_peak",
    "dram__throughput.avg.pct_of_peak_sustained_elapsed": "dram_throughput_pct",
    "sm__throughput.avg.pct_of_peak_sustained_elapsed": "sm_throughput_pct",
    "launch__registers_per_thread": "registers",
    "launch__grid_size": "grid",
    "launch__block_size": "block",
    "sm__warps_active.avg.pct_of_peak_sustained_active": "achieved_occupancy_pct",
    "sm__inst_executed.avg.per_cycle_active": "ipc",
    "smsp__inst_executed.sum": "warp_instructions",
    "l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum": "smem_bank_conflicts",
}


def main(rep):
    raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(raw)))
    h = rows[0]
    units = dict(zip(h, rows[1])) if len(rows) > 1 else {}
    out = []
    for r in rows[2:]:
        d = dict(zip(h, r))
        k = {"kernel": d.get("Kernel Name", "")[:120]}
        for m, name in WANT.items():
            if m in d and d[m] not in ("", "n/a"):
                try:
                    k[name] = float(d[m].replace(",", ""))
                except ValueError:
                    k[name] = d[m]
                if units.get(m):
                    k[name + "_unit"] = units[m]
        stalls = {kk.replace("smsp__pcsamp_warps_issue_stalled_", ""): float(v or 0) for kk, v in d.items()
                  if kk.startswith("smsp__pcsamp_warps_issue_stalled_") and not kk.endswith("not_issued")}
        tot = sum(stalls.values()) or 1.0
        k["top_stalls_pct"] = {a: round(100 * b / tot, 1) for a, b in sorted(stalls.items(), key=lambda x: -x[1])[:6]}
        out.append(k)
    json.dump(out, sys.stdout, indent=1)
    print()


if __name__ == "__main__":
    main(sys.argv[1])
