timeout 300 python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1 || { echo build failed; exit 1; }
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -p no:cacheprovider --timeout 300 -k "host" 2>&1 | tail -3
timeout 400 python bench.py --no-cpu-baseline --no-sc --no-dmma --no-small --no-sp --steps 50 > gpurun_out/e2e_bench.json 2> gpurun_out/e2e_bench.err; python -c "
import json; d=json.load(open('gpurun_out/e2e_bench.json')); print('device', d['ms_per_step'], '%.3e' % d['value'], 'e2e %.3e' % d['e2e']['value'], d['clocks'])"
tail -2 gpurun_out/e2e_bench.err
