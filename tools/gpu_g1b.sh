bash tools/g1run.sh
timeout 300 python -c "import sys; sys.path.insert(0,'.'); from paper_conf_ipps_razakhllknvn24_b200 import build; build.build(force=True)" > /dev/null 2>&1
bash tools/gpu_g1.sh
