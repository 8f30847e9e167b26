# quick check of the GEMM-1 path: build, the int8 / SP / dense / parity tests, a short bench
timeout 300 python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1 || { echo build failed; exit 1; }
timeout 900 python -m pytest tests/test_gpu_i8.py tests/test_gpu_sp.py tests/test_gpu_dense_d.py tests/test_gpu_determinism.py -q -x -p no:cacheprovider --timeout 300 2>&1 | tail -6
timeout 300 python bench.py --no-cpu-baseline --no-e2e --no-sc --no-dmma --no-small --steps 30 > gpurun_out/g1_bench.json 2> gpurun_out/g1_bench.err; python -c "
import json; d=json.load(open('gpurun_out/g1_bench.json')); print('fp64', round(d['ms_per_step'],4), d['clocks'])
for k,v in d['kernels'].items(): print(' ', k, round(v['ms_per_launch'],4), v.get('frac') and round(v['frac'],3))
s=d['sp_mode']; print('sp', round(s['ms_per_step'],4))
for k,v in s['kernels'].items(): print(' ', k, round(v['ms_per_launch'],4), v.get('frac') and round(v['frac'],3))"
tail -3 gpurun_out/g1_bench.err
