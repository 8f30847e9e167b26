#!/bin/bash
# A/B of dens.cu variants tmp_variants/dens_<name>.cu: build, density + SP tests, launch list of the density kernels
set -u
C=paper_conf_ipps_razakhllknvn24_b200/csrc
cp $C/dens.cu /tmp/dens_orig.cu
for v in "$@"; do
  cp tmp_variants/dens_$v.cu $C/dens.cu
  python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1 || { echo "$v build failed"; continue; }
  timeout 300 python -m pytest tests/test_gpu_density.py tests/test_gpu_sp.py -q -x 2>&1 | tail -1
  timeout 180 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/v.csv python bench.py --steps 3 --warmup 1 --no-cpu-baseline --no-e2e --no-sc --no-dmma --no-small > /dev/null 2>&1
  echo "variant $v"; python tools/launches.py gpurun_out/v.csv 2>/dev/null | grep -E "k_density_q"
done
cp /tmp/dens_orig.cu $C/dens.cu
