# GEMM-1 role-wait timing (printf build), then the normal build
LFD_NVCC_DEFINES=-DLFD_G1_TIMING timeout 300 python -c "import sys; sys.path.insert(0,'.'); from paper_conf_ipps_razakhllknvn24_b200 import build; build.build(force=True)" && timeout 120 python tools/fx_timing.py 2 2>&1 | grep "^g1" | tail -8
