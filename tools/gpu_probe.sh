#!/bin/bash
# Probe session: guard-band tests, ncu --set full captures of the named kernels of the C2 bench loop, then the
# role-wait instrumentation build of the fused first factor.  bash tools/gpu_probe.sh TAG "kre1 kre2 ..."
set -u
TAG=${1:-probe}; KRES=${2:-"k_gemm2x_i8 k_density_y"}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/${TAG}_build.log 2>&1 || { tail -30 gpurun_out/${TAG}_build.log; exit 1; }
timeout 600 python -m pytest tests/test_gpu_guard.py -q -x > gpurun_out/${TAG}_guard.log 2>&1; echo "guard rc=$?" >> gpurun_out/${TAG}_guard.log
tail -3 gpurun_out/${TAG}_guard.log
for k in $KRES; do
  timeout 900 ncu --set full --import-source on --clock-control none -k regex:"$k" -s 3 -c 1 -o gpurun_out/${TAG}_$k -f \
    python bench.py --steps 2 --warmup 1 --no-cpu-baseline --no-e2e --no-sc --no-sp --no-dmma --no-small > gpurun_out/${TAG}_${k}_ncu.log 2>&1
  tail -1 gpurun_out/${TAG}_${k}_ncu.log
done
if [ -n "${FXT:-}" ]; then
  LFD_NVCC_DEFINES=-DLFD_FX_TIMING python -c "from paper_conf_ipps_razakhllknvn24_b200 import build as b; b.build(force=True)" > gpurun_out/${TAG}_fxbuild.log 2>&1
  timeout 120 python tools/fx_timing.py 4 > gpurun_out/${TAG}_fxtiming.log 2>&1
  tail -20 gpurun_out/${TAG}_fxtiming.log
fi
ls gpurun_out/
