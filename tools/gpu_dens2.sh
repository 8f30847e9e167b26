#!/bin/bash
# density: tests, cold-L2 probe (32/64/16 active), in-step bench per shape (tuning build), ncu full of the default
set -u
TAG=${1:-dens2}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/${TAG}_build.log 2>&1 || { echo build failed; tail -30 gpurun_out/${TAG}_build.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu_density.py tests/test_gpu_parity.py -q -x > gpurun_out/${TAG}_pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/${TAG}_pytest.log
tail -4 gpurun_out/${TAG}_pytest.log
timeout 300 python tools/dens_probe.py > gpurun_out/${TAG}_probe.jsonl 2>&1; cat gpurun_out/${TAG}_probe.jsonl
timeout 300 python tools/dens_probe.py --sp >> gpurun_out/${TAG}_probe.jsonl 2>&1; tail -3 gpurun_out/${TAG}_probe.jsonl
timeout 600 ncu --set full --import-source on --clock-control none -k regex:"k_density_q" -s 3 -c 1 -o gpurun_out/${TAG}_dq -f \
    python bench.py --steps 2 --warmup 1 --no-cpu-baseline --no-e2e --no-sc --no-sp --no-dmma --no-small > gpurun_out/${TAG}_ncu.log 2>&1
tail -1 gpurun_out/${TAG}_ncu.log
LFD_NVCC_DEFINES=-DLFD_TUNING_KNOBS python -c "from paper_conf_ipps_razakhllknvn24_b200 import build as b; b.build(force=True)" > gpurun_out/${TAG}_tbuild.log 2>&1
for sh in "12 2 2 4 3" "24 1 2 3 2" "36 1 2 3 2" "8 2 2 3 2" "24 1 1 4 3" "72 1 2 3 2" "8 1 2 6 3"; do
  set -- $sh
  LFD_DENS_ZC=$1 LFD_DENS_PX=$2 LFD_DENS_YC=$3 LFD_DENS_OWN=$4 LFD_DENS_XP=$5 timeout 200 python bench.py --no-cpu-baseline --no-e2e --no-sc --no-sp --no-dmma --no-small --steps 50 > gpurun_out/${TAG}_b.json 2>/dev/null
  python -c "
import json; d=json.load(open('gpurun_out/${TAG}_b.json')); k=d['kernels']['density']
print('shape $sh', 'step', round(d['ms_per_step'],4), 'dens', round(k['ms_per_launch'],4), round(k['frac'],3))"
done
