#!/bin/bash
# In-step A/B (no ncu, warm L2 as in the bench) of nl_i8.cu variants tmp_variants/i8_<name>.cu
set -u
C=paper_conf_ipps_razakhllknvn24_b200/csrc
cp $C/nl_i8.cu /tmp/i8_orig.cu
for v in "$@"; do
  cp tmp_variants/i8_$v.cu $C/nl_i8.cu
  python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1 || { echo "$v build failed"; continue; }
  timeout 300 python bench.py --no-cpu-baseline --no-e2e --no-sc --no-dmma --no-small > gpurun_out/v8.json 2>/dev/null
  python -c "
import json; d=json.load(open('gpurun_out/v8.json')); k=d['kernels']
print('$v', round(d['ms_per_step'],4), 'nl_back', round(k['nl_back']['ms_per_launch'],4), 'nl_proj', round(k['nl_proj']['ms_per_launch'],4), 'dens', round(k['density']['ms_per_launch'],4), 'sp', round(d['sp_mode']['ms_per_step'],4))"
done
cp /tmp/i8_orig.cu $C/nl_i8.cu
