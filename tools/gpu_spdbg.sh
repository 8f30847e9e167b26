timeout 300 python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 300 compute-sanitizer --tool memcheck python -m pytest tests/test_gpu_sp.py -q -x -k "int8_digit_gemms and P0" 2>&1 | grep -v "^\s*$" | head -60
