#!/bin/bash
# Build one scan_sweep binary per knob set (scan.cu recompiled with -D flags, the
# other objects from the in-tree build) and run them all.  Build here, run on the GPU:
#   tools/scan_sweep.sh build ; tools/scan_sweep.sh run > gpurun_out/scan_sweep.jsonl
set -e
ROOT=$(cd "$(dirname "$0")/.." && pwd)
OUT=$ROOT/tools/_sweep
CS=$ROOT/paper_conf_pldi_henriksenseho17_b200/csrc
VARIANTS=${VARIANTS:-"R5_STA6_STC4_DA2_TPS4 R7_STA4_STC3_DA2_TPS4 R5_STA6_STC4_DA1_TPS8 R7_STA4_STC3_DA1_TPS4 NC384_R5_STA4_STC3_DA1_TPS4 NC512_R3_STA6_STC4_DA1_TPS4 NC384_R3_STA8_STC4_DA1_TPS8"}
if [ "$1" = build ]; then
  mkdir -p $OUT
  python $ROOT/paper_conf_pldi_henriksenseho17_b200/build.py >/dev/null
  objs=$(ls $ROOT/paper_conf_pldi_henriksenseho17_b200/_build/*.o | grep -v '/scan.o')
  for v in $VARIANTS; do
    flags=""
    for kv in ${v//_/ }; do k=$(echo $kv | sed 's/[0-9]*$//'); val=${kv#$k}
      case $k in X*) flags="$flags -DFS_SCANR_${k#X}=$val";; I*) flags="$flags -DFS_SCAN_IMPL=$val";; *) flags="$flags -DFS_SCANW_$k=$val";; esac; done
    ( nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 --expt-relaxed-constexpr -I$ROOT/include -I$CS $flags \
        -c $CS/scan.cu -o $OUT/scan_$v.o && \
      nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -I$ROOT/include $ROOT/tools/scan_sweep.cu \
        $OUT/scan_$v.o $objs -o $OUT/sweep_$v ) &
  done
  wait
else
  for v in $VARIANTS; do timeout 60 $OUT/sweep_$v $v || echo "{\"tag\": \"$v\", \"failed\": 1}"; done
fi
