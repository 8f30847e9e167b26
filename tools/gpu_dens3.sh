#!/bin/bash
# density (L2 prefetch): tests, cold probe, bench default, launch list, plus the fused-kernel (8 march warps) check
set -u
TAG=${1:-dens3}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/${TAG}_build.log 2>&1 || { echo build failed; tail -30 gpurun_out/${TAG}_build.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu_density.py tests/test_gpu_parity.py tests/test_gpu_i8.py tests/test_gpu_guard.py -q -x > gpurun_out/${TAG}_pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/${TAG}_pytest.log
tail -4 gpurun_out/${TAG}_pytest.log
timeout 300 python tools/dens_probe.py > gpurun_out/${TAG}_probe.jsonl 2>&1; cat gpurun_out/${TAG}_probe.jsonl
timeout 300 python bench.py --no-cpu-baseline --no-e2e --no-sc --no-dmma --no-small --steps 50 > gpurun_out/${TAG}_bench.json 2> gpurun_out/${TAG}_bench.err
python - <<PY
import json
d=json.load(open("gpurun_out/${TAG}_bench.json"))
print("ms/step", round(d["ms_per_step"],4), "value %.3e" % d["value"], d["clocks"])
for k,v in d["kernels"].items(): print(k, round(v["ms_per_launch"],4), v["launches"], round(v["share"],3), v.get("frac"))
sp=d.get("sp_mode") or {}
print("sp", sp.get("ms_per_step"), (sp.get("kernels") or {}).get("density"))
PY
timeout 180 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${TAG}_launches.csv \
   python bench.py --steps 3 --warmup 1 --no-cpu-baseline --no-e2e --no-sc --no-sp --no-dmma --no-small > /dev/null 2>&1
python tools/launches.py gpurun_out/${TAG}_launches.csv 2>/dev/null | head -8
