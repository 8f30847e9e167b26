#!/bin/bash
# GEMM-1 MMA schedules (LFD_G1_WIDE = 0..3): int8 parity tests under each, then a same-box bench A/B.
mkdir -p gpurun_out
for W in 1 2 3; do
  LFD_G1_WIDE=$W timeout 300 python -m pytest tests/test_gpu_i8.py -x -q > gpurun_out/g1s_pytest$W.log 2>&1; echo "wide $W pytest rc=$?"; tail -1 gpurun_out/g1s_pytest$W.log
done
for rep in 1 2; do for W in 0 1 2 3; do
LFD_G1_WIDE=$W timeout 300 python bench.py --no-cpu-baseline --no-e2e --no-sc --no-sp > gpurun_out/g1s_bench$W.json 2> /dev/null
python - <<PY
import json
d=json.load(open("gpurun_out/g1s_bench$W.json")); k=d["kernels"]
print("wide $W ms/step", round(d["ms_per_step"],4), "nl_proj", round(k["nl_proj"]["ms_per_launch"],4), "nl_back", round(k["nl_back"]["ms_per_launch"],4), d["clocks"]["sm_mhz"])
PY
done; done
for W in 0 3; do
LFD_I8_TIMING=1 LFD_G1_WIDE=$W timeout 300 python bench.py --no-cpu-baseline --no-e2e --no-sc --no-sp --steps 10 --warmup 3 > /dev/null 2> gpurun_out/g1s_t$W.err
echo "timing wide $W"; grep "g1 timing" gpurun_out/g1s_t$W.err | tail -1
done
