#!/bin/bash
# A/B of kin.cu variants tmp_variants/kin_<name>.cu: build, parity subset, launch list of the small kernels + in-step bench
set -u
C=paper_conf_ipps_razakhllknvn24_b200/csrc
cp $C/kin.cu /tmp/kin_orig.cu
for v in "$@"; do
  cp tmp_variants/kin_$v.cu $C/kin.cu
  python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1 || { echo "$v build failed"; continue; }
  timeout 300 python -m pytest tests/test_gpu_i8.py tests/test_gpu_sp.py -q -x 2>&1 | tail -1
  timeout 180 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/v.csv python bench.py --steps 3 --warmup 1 --no-cpu-baseline --no-e2e --no-sc --no-dmma --no-small > /dev/null 2>&1
  echo "variant $v"; python tools/launches.py gpurun_out/v.csv 2>/dev/null | grep -E "k_phase|kin_yz"
  timeout 300 python bench.py --no-cpu-baseline --no-e2e --no-sc --no-dmma --no-small > gpurun_out/v9.json 2>/dev/null
  python -c "
import json; d=json.load(open('gpurun_out/v9.json')); k=d['kernels']
print('$v', round(d['ms_per_step'],4), 'phase', round(k['phase']['ms_per_launch'],4), 'sp', round(d['sp_mode']['ms_per_step'],4))"
done
cp /tmp/kin_orig.cu $C/kin.cu
