#!/bin/bash
# full ncu captures (with source) of k_gemm1_i8 and k_density_y in one session
set -u
bash tools/ncu_one.sh r02f_g1 "k_gemm1_i8" 3
timeout 900 ncu --set full --import-source on --clock-control none -k regex:"k_density_y" -s 3 -c 1 -o gpurun_out/r02f_dens -f \
  python bench.py --steps 2 --warmup 1 --no-cpu-baseline --no-e2e --no-sc --no-sp --no-dmma --no-small > gpurun_out/r02f_dens_ncu.log 2>&1
ls -la gpurun_out/*.ncu-rep
