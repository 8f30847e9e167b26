#!/bin/bash
# Density kernel session: build, density + parity tests, quick bench + launch list, then the tuning-knob build
# and the shape sweep.   bash tools/gpu_dens.sh TAG
set -u
TAG=${1:-dens}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/${TAG}_build.log 2>&1 || { echo build failed; tail -30 gpurun_out/${TAG}_build.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu_density.py tests/test_gpu_parity.py tests/test_gpu_sp.py tests/test_gpu_guard.py -q -x > gpurun_out/${TAG}_pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/${TAG}_pytest.log
tail -15 gpurun_out/${TAG}_pytest.log
timeout 300 python bench.py --no-cpu-baseline --no-e2e --no-sc --no-dmma --no-small --steps 50 > gpurun_out/${TAG}_bench.json 2> gpurun_out/${TAG}_bench.err
python - <<PY
import json
d=json.load(open("gpurun_out/${TAG}_bench.json"))
print("ms/step", round(d["ms_per_step"],4), "value %.3e" % d["value"], d["clocks"])
for k,v in d["kernels"].items(): print(k, round(v["ms_per_launch"],4), v["launches"], round(v["share"],3), v.get("frac"))
sp=d.get("sp_mode") or {}
print("sp", sp.get("ms_per_step"), (sp.get("kernels") or {}).get("density"))
PY
tail -3 gpurun_out/${TAG}_bench.err
timeout 180 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${TAG}_launches.csv \
   python bench.py --steps 3 --warmup 1 --no-cpu-baseline --no-e2e --no-sc --no-sp --no-dmma --no-small > /dev/null 2>&1
python tools/launches.py gpurun_out/${TAG}_launches.csv | head -8
LFD_NVCC_DEFINES=-DLFD_TUNING_KNOBS python -c "from paper_conf_ipps_razakhllknvn24_b200 import build as b; b.build(force=True)" > gpurun_out/${TAG}_tbuild.log 2>&1
timeout 600 python tools/dens_sweep.py > gpurun_out/${TAG}_sweep.jsonl 2>&1
sort -t: -k7 -n gpurun_out/${TAG}_sweep.jsonl | head -5
python - <<PY
import json
rows=[json.loads(l) for l in open("gpurun_out/${TAG}_sweep.jsonl") if l.startswith("{")]
rows.sort(key=lambda r: r["ms"])
for r in rows[:12]: print(r)
PY
