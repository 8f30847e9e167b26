#!/bin/bash
# A/B of (nl_fx.cu, nl_i8.cu) variant pairs in tmp_variants/: args "fxname:i8name" ...
set -u
for v in "$@"; do
  fx=${v%%:*}; i8=${v##*:}
  cp tmp_variants/$fx.cu paper_conf_ipps_razakhllknvn24_b200/csrc/nl_fx.cu
  cp tmp_variants/$i8.cu paper_conf_ipps_razakhllknvn24_b200/csrc/nl_i8.cu
  python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1 || { echo "$v build failed"; continue; }
  timeout 200 python -m pytest tests/test_gpu_i8.py tests/test_gpu_sp.py -q -x 2>&1 | tail -1
  timeout 180 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/v.csv python bench.py --steps 3 --warmup 1 --no-cpu-baseline --no-e2e --no-sc --no-dmma --no-small > /dev/null 2>&1
  echo "variant $v"; python tools/launches.py gpurun_out/v.csv | grep -E "gemm2x|gemm2_i8"
done
