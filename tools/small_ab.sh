#!/bin/bash
# Whole GPU suite, then the headline bench twice (small-kernel change check).
mkdir -p gpurun_out
timeout 600 python -m pytest tests -m gpu -x -q > gpurun_out/sm_pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/sm_pytest.log
tail -2 gpurun_out/sm_pytest.log
for rep in 1 2; do
timeout 300 python bench.py --no-cpu-baseline --no-e2e --no-sc --no-sp > gpurun_out/sm_bench$rep.json 2> /dev/null
python - <<PY
import json
d=json.load(open("gpurun_out/sm_bench$rep.json")); k=d["kernels"]
print("ms/step", round(d["ms_per_step"],4), {n: round(v["ms_per_launch"],4) for n, v in k.items() if n in ("nl_carry","nl_norm","nl_reduce","nl_proj")}, d["clocks"]["sm_mhz"])
PY
done
