#!/bin/bash
# Quick gpurun session: build, a subset of GPU tests, bench (no ncu).
# Usage: bash tools/gpu_quick.sh TAG "pytest -k expression or empty" [bench args]
set -u
TAG=${1:-quick}; KEXPR=${2:-}; shift 2 || true
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/${TAG}_build.log 2>&1 || { echo build failed; tail -30 gpurun_out/${TAG}_build.log; exit 1; }
if [ -n "$KEXPR" ]; then
  timeout 900 python -m pytest tests -m gpu -x -q -k "$KEXPR" > gpurun_out/${TAG}_pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/${TAG}_pytest_gpu.log
  tail -4 gpurun_out/${TAG}_pytest_gpu.log
fi
timeout 600 python bench.py --no-cpu-baseline "$@" > gpurun_out/${TAG}_bench.json 2> gpurun_out/${TAG}_bench.err
python - <<PY
import json
d=json.load(open("gpurun_out/${TAG}_bench.json"))
print("ms/step", round(d["ms_per_step"],4), "value %.3e" % d["value"], d["clocks"])
for k,v in d["kernels"].items(): print(k, round(v["ms_per_launch"],4), v["launches"], round(v["share"],3), v.get("frac"))
print("e2e", d["e2e"] and "%.3e" % d["e2e"]["value"], "seq", d.get("sequence_mode") and round(d["sequence_mode"]["ms_per_step"],4))
PY
