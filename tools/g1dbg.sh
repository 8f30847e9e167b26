python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for D in 0 1 4 8 12 13; do
LFD_I8_DBG1=$D timeout 300 python bench.py --no-cpu-baseline --no-e2e --no-sc --no-sp > gpurun_out/g1dbg$D.json 2>/dev/null
python -c "
import json; d=json.load(open('gpurun_out/g1dbg$D.json')); print('dbg1 $D nl_proj', round(d['kernels']['nl_proj']['ms_per_launch'],4))"
done
