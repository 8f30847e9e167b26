timeout 300 python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 900 python -m pytest tests/test_gpu_sp.py -q -p no:cacheprovider --timeout 240 2>&1 | tail -8
timeout 300 python bench.py --no-cpu-baseline --no-e2e --no-sc --no-dmma --no-small --steps 30 > gpurun_out/spi8_bench.json 2> gpurun_out/spi8_bench.err; python -c "
import json; d=json.load(open('gpurun_out/spi8_bench.json')); s=d['sp_mode']; print('fp64', d['ms_per_step'], 'sp', s.get('ms_per_step'), s.get('error'), s.get('nl_path'))
for k,v in s.get('kernels',{}).items(): print(k, v)"
tail -3 gpurun_out/spi8_bench.err
cuobjdump -sass paper_conf_ipps_razakhllknvn24_b200/*.so 2>/dev/null | grep -c UTCIMMA
