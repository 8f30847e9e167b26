timeout 300 python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1 || { echo build failed; exit 1; }
timeout 900 python -m pytest tests/test_gpu_sp.py tests/test_gpu_dense_d.py tests/test_gpu_parity.py -q -x -p no:cacheprovider --timeout 300 2>&1 | tail -4
timeout 300 python bench.py --no-cpu-baseline --no-e2e --no-sc --no-dmma --no-small --steps 30 > gpurun_out/spyz_bench.json 2> gpurun_out/spyz_bench.err; python -c "
import json; d=json.load(open('gpurun_out/spyz_bench.json')); print('fp64', round(d['ms_per_step'],4)); s=d['sp_mode']; print('sp', round(s['ms_per_step'],4), s.get('nl_path'))
for k,v in s['kernels'].items(): print(' ', k, round(v['ms_per_launch'],4), v.get('frac') and round(v['frac'],3))"
tail -2 gpurun_out/spyz_bench.err
