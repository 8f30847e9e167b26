#!/bin/bash
# A/B: each arg "d:f:i" picks tmp_variants/dens_d.cu, nl_fx_f.cu, nl_i8_i.cu
set -u
C=paper_conf_ipps_razakhllknvn24_b200/csrc
for v in "$@"; do
  IFS=: read d f i <<< "$v"
  cp tmp_variants/dens_$d.cu $C/dens.cu; cp tmp_variants/nl_fx_$f.cu $C/nl_fx.cu; cp tmp_variants/nl_i8_$i.cu $C/nl_i8.cu
  python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1 || { echo "$v build failed"; continue; }
  timeout 300 python -m pytest tests/test_gpu_i8.py tests/test_gpu_density.py -q -x 2>&1 | tail -1
  timeout 180 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/v.csv python bench.py --steps 3 --warmup 1 --no-cpu-baseline --no-e2e --no-sc --no-dmma --no-small > /dev/null 2>&1
  echo "variant $v"; python tools/launches.py gpurun_out/v.csv | grep -E "gemm2x|gemm2_i8|density_q"
done
