#!/bin/bash
# ncu --set full of ONE launch of the kernels matching $1 inside `bench.py --only $2`
# usage (on the GPU box): tools/ncu_one.sh <kernel-regex> <primitive[,primitive]> <out-name> [count]
ncu --set full --clock-control none --import-source on -k "regex:$1" -c "${4:-1}" -o "gpurun_out/$3" \
    python bench.py --only "$2" --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > "gpurun_out/$3.log" 2>&1
