#!/bin/bash
# Round-end style session: build, all GPU tests, smoke, the default bench, the ncu launch list, and one
# ncu --set full capture of each main C2 kernel (for profiles/latest_ncu_full_summary.csv).  bash tools/gpu_final.sh TAG
set -u
TAG=${1:-final}
bash tools/gpu_round.sh $TAG
for k in k_gemm2x_i8 k_gemm2_i8 k_kin_yz k_gemm1_i8 k_density_q; do
  timeout 600 ncu --set full --import-source on --clock-control none -k regex:"$k" -s 2 -c 1 -o gpurun_out/${TAG}_full_$k -f \
    python bench.py --steps 2 --warmup 1 --no-cpu-baseline --no-e2e --no-sc --no-sp --no-dmma --no-small > gpurun_out/${TAG}_full_$k.log 2>&1
  tail -1 gpurun_out/${TAG}_full_$k.log
done
ls gpurun_out | grep $TAG
