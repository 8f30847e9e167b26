#!/bin/bash
# A/B of nl_i8.cu variants tmp_variants/i8_<name>.cu: build, SP + i8 tests, launch list of the i8 GEMMs
set -u
C=paper_conf_ipps_razakhllknvn24_b200/csrc
cp $C/nl_i8.cu /tmp/i8_orig.cu
for v in "$@"; do
  cp tmp_variants/i8_$v.cu $C/nl_i8.cu
  python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1 || { echo "$v build failed"; continue; }
  timeout 300 python -m pytest tests/test_gpu_sp.py tests/test_gpu_i8.py tests/test_gpu_guard.py -q -x 2>&1 | tail -1
  timeout 180 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/v.csv python bench.py --steps 3 --warmup 1 --no-cpu-baseline --no-e2e --no-sc --no-dmma --no-small > /dev/null 2>&1
  echo "variant $v"; python tools/launches.py gpurun_out/v.csv | grep -E "gemm[12]_i8"
done
cp /tmp/i8_orig.cu $C/nl_i8.cu
