#!/bin/bash
# GEMM-1 change check: whole GPU suite, then the headline bench twice and the role timing.
mkdir -p gpurun_out
timeout 600 python -m pytest tests -m gpu -x -q > gpurun_out/g1c_pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/g1c_pytest.log
tail -2 gpurun_out/g1c_pytest.log
for rep in 1 2; do
timeout 300 python bench.py --no-cpu-baseline --no-e2e --no-sc --no-sp > gpurun_out/g1c_bench$rep.json 2> /dev/null
python - <<PY
import json
d=json.load(open("gpurun_out/g1c_bench$rep.json")); k=d["kernels"]
print("ms/step", round(d["ms_per_step"],4), "nl_proj", round(k["nl_proj"]["ms_per_launch"],4), "nl_back", round(k["nl_back"]["ms_per_launch"],4), d["clocks"]["sm_mhz"])
PY
done
LFD_I8_TIMING=1 timeout 300 python bench.py --no-cpu-baseline --no-e2e --no-sc --no-sp --steps 10 --warmup 3 > /dev/null 2> gpurun_out/g1c_t.err
grep "g1 timing" gpurun_out/g1c_t.err | tail -1
