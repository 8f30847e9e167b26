#!/bin/bash
# One gpurun session of round 2: build, GPU tests (with durations), smoke, bench, ncu launch list.
# Usage (repo root, under gpurun): bash tools/gpu_round.sh TAG [pytest-args...]
set -u
TAG=${1:-r02}; shift || true
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > gpurun_out/${TAG}_smi.txt 2>&1
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/${TAG}_build.log 2>&1 || { echo build failed; tail -30 gpurun_out/${TAG}_build.log; exit 1; }
timeout 1800 python -m pytest tests -m gpu -q -rA --durations=40 -s "$@" > gpurun_out/${TAG}_pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/${TAG}_pytest_gpu.log
tail -5 gpurun_out/${TAG}_pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/${TAG}_smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/${TAG}_smoke.log
tail -2 gpurun_out/${TAG}_smoke.log
timeout 600 python bench.py > gpurun_out/${TAG}_bench.json 2> gpurun_out/${TAG}_bench.err
python - <<PY
import json
d=json.load(open("gpurun_out/${TAG}_bench.json"))
print("ms/step", round(d["ms_per_step"],4), "value %.3e" % d["value"], d["clocks"])
for k,v in d["kernels"].items(): print(k, round(v["ms_per_launch"],4), v["launches"], round(v["share"],3), v.get("frac"))
print("e2e", d["e2e"] and "%.3e" % d["e2e"]["value"], "dmma", d.get("nl_dmma_mode") and d["nl_dmma_mode"].get("ms_per_step"))
print("small", json.dumps(d.get("other_configs"))[:600])
PY
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${TAG}_launches.csv \
   python bench.py --steps 3 --warmup 1 --no-cpu-baseline --no-e2e --no-sc --no-sp --no-dmma --no-small > gpurun_out/${TAG}_ncu_bench.log 2>&1
echo done
