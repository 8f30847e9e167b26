python -c "import __graft_entry__ as g; g.build()" > gpurun_out/i8b_build.log 2>&1
timeout 300 python tools/i8_check.py P0 C1 C2 > gpurun_out/i8b.log 2>&1; echo rc=$? >> gpurun_out/i8b.log
LFD_NL_I8=1 timeout 300 python bench.py --no-cpu-baseline --no-e2e --no-sc --no-sp > gpurun_out/i8b_bench.json 2> gpurun_out/i8b_bench.err
LFD_NL_I8=1 timeout 300 ncu --set full --clock-control none --import-source on -k regex:k_gemm2_i8 -s 4 -c 1 -o gpurun_out/i8b_prof -f python bench.py --steps 2 --warmup 1 --no-cpu-baseline --no-e2e --no-sc --no-sp > gpurun_out/i8b_ncu.log 2>&1
cat gpurun_out/i8b.log
python - <<'PY'
import json
d=json.load(open("gpurun_out/i8b_bench.json"))
print("ms/step", round(d["ms_per_step"],4))
for k,v in d["kernels"].items(): print(k, round(v["ms_per_launch"],4), v["launches"], round(v["share"],3), v.get("frac"))
PY
