#!/bin/bash
# A/B of (nl_i8.cu, kin.cu) variant pairs in tmp_variants/: args "i8name:kinname" ...
set -u
for v in "$@"; do
  a=${v%%:*}; b=${v##*:}
  cp tmp_variants/$a.cu paper_conf_ipps_razakhllknvn24_b200/csrc/nl_i8.cu
  cp tmp_variants/$b.cu paper_conf_ipps_razakhllknvn24_b200/csrc/kin.cu
  python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1 || { echo "$v build failed"; continue; }
  timeout 300 python -m pytest tests/test_gpu_i8.py tests/test_gpu_parity.py -q -x 2>&1 | tail -1
  timeout 180 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/v.csv python bench.py --steps 3 --warmup 1 --no-cpu-baseline --no-e2e --no-sc --no-dmma --no-small > /dev/null 2>&1
  echo "variant $v"; python tools/launches.py gpurun_out/v.csv | grep -E "gemm1_i8|kin_yz"
done
