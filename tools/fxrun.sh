# (every step bounded by its own timeout: a hang must not eat the gpurun limit)
LFD_NVCC_DEFINES=-DLFD_FX_TIMING timeout 300 python -c "import sys; sys.path.insert(0,'.'); from paper_conf_ipps_razakhllknvn24_b200 import build; build.build(force=True)" && timeout 60 python tools/fx_timing.py 2 2>&1 | tail -8
timeout 300 python -c "import sys; sys.path.insert(0,'.'); from paper_conf_ipps_razakhllknvn24_b200 import build; build.build(force=True)"
timeout 900 bash tools/gpu_fx.sh fx3 tests/test_gpu_i8.py
