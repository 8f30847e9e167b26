#!/bin/bash
# ncu --set full capture of one SP (complex64) kernel of the bench's SP mode.  bash tools/ncu_sp.sh TAG DEMANGLED_REGEX
set -u
TAG=$1; KRE=$2; CNT=${3:-1}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/${TAG}_build.log 2>&1 || { tail -20 gpurun_out/${TAG}_build.log; exit 1; }
timeout 300 python -m pytest tests/test_gpu_sp.py tests/test_gpu_i8.py -q -x 2>&1 | tail -1
timeout 900 ncu --set full --import-source on --clock-control none --kernel-name-base demangled -k regex:"$KRE" -s 3 -c $CNT -o gpurun_out/${TAG} -f \
  python bench.py --steps 2 --warmup 1 --no-cpu-baseline --no-e2e --no-sc --no-dmma --no-small > gpurun_out/${TAG}_ncu.log 2>&1
tail -3 gpurun_out/${TAG}_ncu.log
ls -la gpurun_out/${TAG}.ncu-rep
