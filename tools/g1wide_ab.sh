#!/bin/bash
# GEMM-1 wide-N schedule: i8 parity tests, then an A/B of LFD_G1_WIDE on one box (bench, headline C2 only).
set -u
mkdir -p gpurun_out
timeout 600 python -m pytest tests -m gpu -x -q > gpurun_out/g1w_pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/g1w_pytest.log
tail -3 gpurun_out/g1w_pytest.log
for W in 0 1 0 1; do
LFD_G1_WIDE=$W timeout 300 python bench.py --no-cpu-baseline --no-e2e --no-sc --no-sp > gpurun_out/g1w_bench$W.json 2> gpurun_out/g1w_bench.err
python - <<PY
import json
d=json.load(open("gpurun_out/g1w_bench$W.json"))
k=d["kernels"]
print("wide $W ms/step", round(d["ms_per_step"],4), "nl_proj", round(k["nl_proj"]["ms_per_launch"],4), "nl_back", round(k["nl_back"]["ms_per_launch"],4), d["clocks"]["sm_mhz"])
PY
done
