#!/bin/bash
# A/B of nl_fx.cu variants tmp_variants/fx_<name>.cu: build, i8 tests, launch list
set -u
C=paper_conf_ipps_razakhllknvn24_b200/csrc
for v in "$@"; do
  cp tmp_variants/fx_$v.cu $C/nl_fx.cu
  python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1 || { echo "$v build failed"; continue; }
  timeout 200 python -m pytest tests/test_gpu_i8.py -q -x 2>&1 | tail -1
  timeout 180 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/v.csv python bench.py --steps 3 --warmup 1 --no-cpu-baseline --no-e2e --no-sc --no-dmma --no-small > /dev/null 2>&1
  echo "variant $v"; python tools/launches.py gpurun_out/v.csv | grep -E "gemm2x"
done
