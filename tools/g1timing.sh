#!/bin/bash
# GEMM-1 role-wait cycles (LFD_I8_TIMING) under the MMA schedules given (default: 0 and 1).
mkdir -p gpurun_out
for W in ${SCHEDS:-0 1}; do
LFD_I8_TIMING=1 LFD_G1_WIDE=$W timeout 300 python bench.py --no-cpu-baseline --no-e2e --no-sc --no-sp --steps 20 --warmup 3 > gpurun_out/g1t_bench$W.json 2> gpurun_out/g1t_$W.err
echo "wide $W"; grep "g1 timing" gpurun_out/g1t_$W.err | tail -1
done
