#!/bin/bash
# GEMM-1: suspend-time hint on the A-buffer waits (LFD_G1_SLEEP) x MMA schedule (LFD_G1_WIDE), same box.
mkdir -p gpurun_out
LFD_G1_SLEEP=1 LFD_G1_WIDE=1 timeout 300 python -m pytest tests/test_gpu_i8.py -x -q 2>&1 | tail -1
for rep in 1 2; do for SW in "0 1" "1 1" "0 0" "1 0"; do set -- $SW
LFD_G1_SLEEP=$1 LFD_G1_WIDE=$2 timeout 300 python bench.py --no-cpu-baseline --no-e2e --no-sc --no-sp > gpurun_out/g1sl.json 2> /dev/null
python - <<PY
import json
d=json.load(open("gpurun_out/g1sl.json")); k=d["kernels"]
print("sleep $1 wide $2 ms/step", round(d["ms_per_step"],4), "nl_proj", round(k["nl_proj"]["ms_per_launch"],4), d["clocks"]["sm_mhz"])
PY
done; done
