#!/bin/bash
# A/B of nl_fx.cu variants in tmp_variants/*.cu (each: build, the i8 tests, ncu launch list of the bench)
set -u
for v in "$@"; do
  cp tmp_variants/$v.cu paper_conf_ipps_razakhllknvn24_b200/csrc/nl_fx.cu
  python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1 || { echo "$v build failed"; continue; }
  timeout 200 python -m pytest tests/test_gpu_i8.py tests/test_gpu_sp.py -q -x 2>&1 | tail -1
  timeout 180 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/v_$v.csv python bench.py --steps 3 --warmup 1 --no-cpu-baseline --no-e2e --no-sc --no-dmma --no-small > /dev/null 2>&1
  echo "variant $v"; python tools/launches.py gpurun_out/v_$v.csv | grep gemm2x
done
