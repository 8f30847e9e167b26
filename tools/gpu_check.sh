#!/bin/bash
# One gpurun session: build, GPU tests, smoke, bench, ncu launch list + full capture of the top kernels
# (FP64 step, SP variant, self-consistent step).
# Usage (from the repo root, under gpurun): bash tools/gpu_check.sh [tag]
set -u
TAG=${1:-r01}
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > gpurun_out/${TAG}_smi.txt 2>&1
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/${TAG}_build.log 2>&1
timeout 1200 python -m pytest tests -m gpu -q > gpurun_out/${TAG}_pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/${TAG}_pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/${TAG}_smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/${TAG}_smoke.log
timeout 600 python bench.py > gpurun_out/${TAG}_bench.json 2> gpurun_out/${TAG}_bench.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${TAG}_launches.csv \
   python bench.py --steps 3 --warmup 1 --no-cpu-baseline --no-e2e --no-sc --no-sp > gpurun_out/${TAG}_ncu_bench.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"${KREGEX:-k_gemm1|k_gemm2|k_kin|k_density}" -s ${KSKIP:-8} -c ${KCOUNT:-6} \
   -o gpurun_out/${TAG}_prof -f python bench.py --steps 2 --warmup 1 --no-cpu-baseline --no-e2e --no-sc --no-sp > gpurun_out/${TAG}_ncu_full.log 2>&1
timeout 600 ncu --set full --clock-control none -k regex:"k_gemm1_sp|k_gemm2_sp|k_kin|k_density" -s 6 -c 5 \
   -o gpurun_out/${TAG}_sp_prof -f python tools/tune.py --knob X --values 0 --steps 2 --sp > gpurun_out/${TAG}_ncu_sp.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${TAG}_sc_launches.csv \
   python tools/sc_bench.py --steps 2 > gpurun_out/${TAG}_ncu_sc.log 2>&1
echo done
