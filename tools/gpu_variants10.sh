#!/bin/bash
# In-step A/B (warm L2, bench timing) of nl_fx.cu variants tmp_variants/fx_<name>.cu, with the i8 parity tests
set -u
C=paper_conf_ipps_razakhllknvn24_b200/csrc
cp $C/nl_fx.cu /tmp/fx_orig.cu
for v in "$@"; do
  cp tmp_variants/fx_$v.cu $C/nl_fx.cu
  python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1 || { echo "$v build failed"; continue; }
  timeout 200 python -m pytest tests/test_gpu_i8.py tests/test_gpu_sp.py -q -x 2>&1 | tail -1
  timeout 300 python bench.py --no-cpu-baseline --no-e2e --no-sc --no-dmma --no-small > gpurun_out/v10.json 2>/dev/null
  python -c "
import json; d=json.load(open('gpurun_out/v10.json')); k=d['kernels']
print('$v', round(d['ms_per_step'],4), 'fx', round(k['nl_back_x']['ms_per_launch'],4), 'kin_yz', round(k['kin_yz']['ms_per_launch'],4), 'sp', round(d['sp_mode']['ms_per_step'],4))"
done
cp /tmp/fx_orig.cu $C/nl_fx.cu
