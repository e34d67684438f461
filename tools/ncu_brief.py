#!/usr/bin/env python
"""One-screen digest of an ncu --set full report: time, DRAM, issue, L1 wavefronts by op,
top stall reasons and the hottest SASS lines (by warp-stall samples).

    python tools/ncu_brief.py gpurun_out/<name>.ncu-rep [n_lines]
"""
import csv
import io
import subprocess
import sys


def raw(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    return [dict(zip(rows[0], r)) for r in rows[2:]]


KEYS = ["gpu__time_duration.sum", "dram__throughput.avg.pct_of_peak_sustained_elapsed",
        "sm__inst_issued.avg.pct_of_peak_sustained_active", "l1tex__throughput.avg.pct_of_peak_sustained_active",
        "smsp__inst_executed.sum", "sm__warps_active.avg.pct_of_peak_sustained_active",
        "l1tex__data_pipe_lsu_wavefronts_mem_shared_op_ld.sum", "l1tex__data_pipe_lsu_wavefronts_mem_shared_op_st.sum",
        "l1tex__data_pipe_lsu_wavefronts_mem_shared_op_atom.sum", "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum",
        "l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum", "launch__registers_per_thread"]


def main(rep, nlines=25):
    for k in raw(rep):
        print(k.get("Kernel Name", "")[:110])
        for key in KEYS:
            print(f"  {key:70s} {k.get(key, '')}")
        st = {n: float(v) for n, v in k.items()
              if n.startswith("smsp__average_warps_issue_stalled_") and n.endswith("_per_issue_active.ratio") and v}
        top = sorted(st.items(), key=lambda t: -t[1])[:8]
        print("  stalls/issue:", ", ".join(f"{n[len('smsp__average_warps_issue_stalled_'):-len('_per_issue_active.ratio')]}={v:.2f}" for n, v in top))
    out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                         capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr = next(i for i, r in enumerate(rows) if r and r[0] == "Address")
    h = rows[hdr]
    ix = {n: i for i, n in enumerate(h)}

    def f(r, n):
        try:
            return float(r[ix[n]].replace(",", ""))
        except (KeyError, ValueError, IndexError):
            return 0.0
    data = [r for r in rows[hdr + 1:] if len(r) == len(h)]
    tot = sum(f(r, "Warp Stall Sampling (All Samples)") for r in data) or 1
    print(f"hot SASS (share of {int(tot)} stall samples; exec count; L1 shared wavefronts):")
    for r in sorted(data, key=lambda r: -f(r, "Warp Stall Sampling (All Samples)"))[:nlines]:
        print(f"  {100 * f(r, 'Warp Stall Sampling (All Samples)') / tot:5.1f}%  {r[ix['Source']][:58]:58s} "
              f"{int(f(r, 'Instructions Executed')):>10d} {int(f(r, 'L1 Wavefronts Shared')):>10d}")


if __name__ == "__main__":
    main(sys.argv[1], int(sys.argv[2]) if len(sys.argv) > 2 else 25)
