#!/bin/bash
# ncu full capture of the density kernel in the C2 step, and the C5 sweep on HEAD
set -u
TAG=${1:-meas}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/${TAG}_build.log 2>&1 || { tail -30 gpurun_out/${TAG}_build.log; exit 1; }
timeout 600 ncu --set full --import-source on --clock-control none -k regex:"k_density_q" -s 3 -c 1 -o gpurun_out/${TAG}_dq -f \
    python bench.py --steps 2 --warmup 1 --no-cpu-baseline --no-e2e --no-sc --no-sp --no-dmma --no-small > gpurun_out/${TAG}_ncu.log 2>&1
tail -1 gpurun_out/${TAG}_ncu.log
timeout 1200 python bench.py --config C5 --steps 5 --warmup 2 > gpurun_out/${TAG}_c5.jsonl 2> gpurun_out/${TAG}_c5.err
tail -2 gpurun_out/${TAG}_c5.err; wc -l gpurun_out/${TAG}_c5.jsonl
