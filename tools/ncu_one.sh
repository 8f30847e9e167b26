#!/bin/bash
# ncu --set full capture (with source) of one kernel of the C2 bench loop.  bash tools/ncu_one.sh TAG KREGEX [SKIP]
set -u
TAG=$1; KRE=$2; SKIP=${3:-3}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/${TAG}_build.log 2>&1 || { tail -20 gpurun_out/${TAG}_build.log; exit 1; }
timeout 900 ncu --set full --import-source on --clock-control none -k regex:"$KRE" -s $SKIP -c 1 -o gpurun_out/${TAG} -f \
  python bench.py --steps 2 --warmup 1 --no-cpu-baseline --no-e2e --no-sc --no-sp --no-dmma --no-small > gpurun_out/${TAG}_ncu.log 2>&1
tail -3 gpurun_out/${TAG}_ncu.log
ls -la gpurun_out/${TAG}.ncu-rep
