#!/bin/bash
# A/B of the SP unroll factors: tmp_variants/kin_<x>.cu + i8_<x>.cu together
set -u
C=paper_conf_ipps_razakhllknvn24_b200/csrc
cp $C/kin.cu /tmp/kin_orig.cu; cp $C/nl_i8.cu /tmp/i8_orig.cu
for v in "$@"; do
  cp tmp_variants/kin_$v.cu $C/kin.cu; cp tmp_variants/i8_$v.cu $C/nl_i8.cu
  python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1 || { echo "$v build failed"; continue; }
  timeout 300 python -m pytest tests/test_gpu_sp.py -q -x 2>&1 | tail -1
  timeout 180 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/v.csv python bench.py --steps 3 --warmup 1 --no-cpu-baseline --no-e2e --no-sc --no-dmma --no-small > /dev/null 2>&1
  echo "variant $v"; python tools/launches.py gpurun_out/v.csv | grep -E "float2"
done
cp /tmp/kin_orig.cu $C/kin.cu; cp /tmp/i8_orig.cu $C/nl_i8.cu
