#!/bin/bash
# in-step density per (shape, L2 prefetch depth), tuning build; args "zc px nyc nso nsx pf"
set -u
TAG=${1:-dens7}; shift
mkdir -p gpurun_out
LFD_NVCC_DEFINES=-DLFD_TUNING_KNOBS python -c "from paper_conf_ipps_razakhllknvn24_b200 import build as b; b.build(force=True)" > gpurun_out/${TAG}_tbuild.log 2>&1 || { tail gpurun_out/${TAG}_tbuild.log; exit 1; }
for sh in "$@"; do
  set -- $sh
  LFD_DENS_ZC=$1 LFD_DENS_PX=$2 LFD_DENS_YC=$3 LFD_DENS_OWN=$4 LFD_DENS_XP=$5 timeout 200 python bench.py --no-cpu-baseline --no-e2e --no-sc --no-dmma --no-small --steps 30 --warmup 5 > gpurun_out/${TAG}_b.json 2>/dev/null
  python -c "
import json; d=json.load(open('gpurun_out/${TAG}_b.json')); k=d['kernels']['density']; s=d['sp_mode']; ks=s['kernels']['density']
print('shape+pf $sh', 'fp64 step', round(d['ms_per_step'],4), 'dens', round(k['ms_per_launch'],4), '| sp step', round(s['ms_per_step'],4), 'dens', round(ks['ms_per_launch'],4))"
done
