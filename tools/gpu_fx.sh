#!/bin/bash
# quick check of a kernel change: build, one GPU test file (bounded), then the bench (no extras) and a launch list
set -u
TAG=${1:-fx}; TESTS=${2:-tests/test_gpu_i8.py}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/${TAG}_build.log 2>&1 || { echo build failed; tail -30 gpurun_out/${TAG}_build.log; exit 1; }
timeout 300 python -m pytest $TESTS -x -q -s > gpurun_out/${TAG}_pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/${TAG}_pytest.log
tail -15 gpurun_out/${TAG}_pytest.log
timeout 120 python bench.py --no-cpu-baseline --no-e2e --no-sc --no-sp --no-dmma --no-small --steps 50 > gpurun_out/${TAG}_bench.json 2> gpurun_out/${TAG}_bench.err
python - <<PY
import json
d=json.load(open("gpurun_out/${TAG}_bench.json"))
print("ms/step", round(d["ms_per_step"],4), "value %.3e" % d["value"], d["clocks"])
for k,v in d["kernels"].items(): print(k, round(v["ms_per_launch"],4), v["launches"], round(v["share"],3), v.get("frac"))
PY
tail -3 gpurun_out/${TAG}_bench.err
timeout 180 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${TAG}_launches.csv \
   python bench.py --steps 3 --warmup 1 --no-cpu-baseline --no-e2e --no-sc --no-sp --no-dmma --no-small > /dev/null 2>&1
python tools/launches.py gpurun_out/${TAG}_launches.csv | head -12
