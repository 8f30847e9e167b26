#!/bin/bash
# build, a GPU test subset, bench (no extras), launch list
set -u
TAG=${1:-q}; TESTS=${2:-"tests/test_gpu_parity.py tests/test_gpu_i8.py tests/test_gpu_density.py"}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/${TAG}_build.log 2>&1 || { echo build failed; tail -30 gpurun_out/${TAG}_build.log; exit 1; }
timeout 900 python -m pytest $TESTS -q -x > gpurun_out/${TAG}_pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/${TAG}_pytest.log
tail -3 gpurun_out/${TAG}_pytest.log
timeout 300 python bench.py --no-cpu-baseline --no-sc --no-dmma --no-small --steps 50 > gpurun_out/${TAG}_bench.json 2> gpurun_out/${TAG}_bench.err
python - <<PY
import json
d=json.load(open("gpurun_out/${TAG}_bench.json"))
print("ms/step", round(d["ms_per_step"],4), "value %.3e" % d["value"], d["clocks"], "launches", d["gpu_launches"])
for k,v in d["kernels"].items(): print(k, round(v["ms_per_launch"],4), v["launches"], round(v["share"],3), v.get("frac"))
sp=d.get("sp_mode") or {}
print("e2e %.3e" % d["e2e"]["value"], "sp", sp.get("ms_per_step"), "seq", (d.get("sequence_mode") or {}).get("ms_per_step"))
PY
tail -2 gpurun_out/${TAG}_bench.err
timeout 180 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${TAG}_launches.csv \
   python bench.py --steps 3 --warmup 1 --no-cpu-baseline --no-e2e --no-sc --no-sp --no-dmma --no-small > /dev/null 2>&1
python tools/launches.py gpurun_out/${TAG}_launches.csv 2>/dev/null | head -14
