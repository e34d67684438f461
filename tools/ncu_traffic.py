#!/usr/bin/env python
"""Summarise an ncu launch list of bench.py (gpu__time_duration.sum,
dram__bytes_read.sum, dram__bytes_write.sum per launch) per hot-path primitive.

Every primitive of a bench step launches exactly one libfutseg kernel, in the
fixed step order, so the fs:: launches are assigned to primitives cyclically.

    python tools/ncu_traffic.py gpurun_out/launches.csv > profiles/ncu_traffic.json
"""
import csv
import json
import sys

ORDER = ["redomap_f32_add", "nn_argmin_redomap", "scanomap_f32_add", "stream_red_kmeans_k32_d34",
         "seg_reduce_row_L32", "seg_reduce_row_L1024", "seg_reduce_row_L65536", "seg_reduce_row_L1048576",
         "seg_reduce_col_L1024", "seg_scan_row_L1024", "transpose_2d_f32"]


def main(path):
    rows = list(csv.reader(open(path)))
    hi = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
    h = rows[hi]
    ki, mi, vi, ii = h.index("Kernel Name"), h.index("Metric Name"), h.index("Metric Value"), h.index("ID")
    launches = {}
    for r in rows[hi + 1:]:
        if len(r) <= vi:
            continue
        d = launches.setdefault(int(r[ii]), {"kernel": r[ki]})
        d[r[mi]] = float(r[vi].replace(",", ""))
    ours = [launches[i] for i in sorted(launches) if "fs::" in launches[i]["kernel"]]
    per = {}
    for j, L in enumerate(ours):
        name = ORDER[j % len(ORDER)]
        e = per.setdefault(name, {"kernel": L["kernel"].split("(")[0], "launches": 0, "ns": [], "traffic": []})
        e["launches"] += 1
        e["ns"].append(L.get("gpu__time_duration.sum"))
        e["traffic"].append(L.get("dram__bytes_read.sum", 0) + L.get("dram__bytes_write.sum", 0))
    out = {}
    for k, e in per.items():
        out[k] = {"kernel": e["kernel"], "launches": e["launches"],
                  "ncu_ms_avg": round(sum(e["ns"]) / len(e["ns"]) / 1e6, 4),
                  "traffic_bytes_per_launch": int(sum(e["traffic"]) / len(e["traffic"]))}
    tot = sum(v["ncu_ms_avg"] for v in out.values())
    for v in out.values():
        v["share_of_step"] = round(v["ncu_ms_avg"] / tot, 4)
    json.dump(out, sys.stdout, indent=1)
    print()


if __name__ == "__main__":
    main(sys.argv[1])
