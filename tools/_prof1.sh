set -x
python paper_conf_pldi_henriksenseho17_b200/build.py > /dev/null 2>&1
for c in "scanomap" "seg_scan 3" "seg_scan 33" "seg_scan 1000" "seg_scan 2097152" "seg_scan 524288" "seg_scan 65537 col" "seg_scan 3 col" "seg_scan 2 col" "seg_scan 7 col" "seg_scan 134217728 col"; do python tools/prof_case.py $c; done > gpurun_out/prof1.txt 2>&1
ncu --set full --clock-control none --import-source on -k "regex:scan_ws_kernel" -s 2 -c 1 -o gpurun_out/scanw python tools/prof_case.py scanomap > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k "regex:rows" -s 2 -c 1 -o gpurun_out/ks3 python tools/prof_case.py seg_scan 1000 > /dev/null 2>&1
