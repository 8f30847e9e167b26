python -c "import __graft_entry__ as g; g.build()" > gpurun_out/i8c_build.log 2>&1
for D in ${DBGS:-0 1 2 3}; do
LFD_I8_DBG=$D LFD_NL_I8=1 timeout 300 python bench.py --no-cpu-baseline --no-e2e --no-sc --no-sp > gpurun_out/i8c_bench$D.json 2> gpurun_out/i8c_bench.err
python - <<PY
import json
d=json.load(open("gpurun_out/i8c_bench$D.json"))
print("dbg $D ms/step", round(d["ms_per_step"],4), "nl_back", round(d["kernels"]["nl_back"]["ms_per_launch"],4))
PY
done
