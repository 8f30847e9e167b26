timeout 300 python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 600 python -m pytest tests/test_gpu_sanitizer.py -q -k "i8" 2>&1 | tail -3
timeout 900 bash tools/fxrun.sh
