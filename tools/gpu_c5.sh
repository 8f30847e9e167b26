#!/bin/bash
# C5 sweep on HEAD + the narrow-tile parity tests
set -u
mkdir -p gpurun_out
timeout 300 python -c "import __graft_entry__ as g; g.build()" > gpurun_out/c5_build.log 2>&1 || { tail -20 gpurun_out/c5_build.log; exit 1; }
timeout 600 python -m pytest tests/test_gpu_parity.py -q -k "narrow or ragged or c2_full" > gpurun_out/c5_pytest.log 2>&1; tail -2 gpurun_out/c5_pytest.log
timeout 1500 python bench.py --config C5 --steps 3 --warmup 1 > gpurun_out/r02_c5.jsonl 2> gpurun_out/r02_c5.err; tail -3 gpurun_out/r02_c5.err
python - <<'PY'
import json
for l in open("gpurun_out/r02_c5.jsonl"):
    r=json.loads(l); c=r["config"]
    print(c["norb"], c["nproj"], r["path"][:10], "g1 %.1f TF (%.2f)" % (r["gemm1"]["fp64_equiv_tflops"], r["gemm1"]["frac_of_fp64_dmma_peak"]),
          "g2 %.1f TF (%.2f)" % (r["gemm2"]["fp64_equiv_tflops"], r["gemm2"]["frac_of_fp64_dmma_peak"]), "acc %.1e" % r["update_rel_error_vs_cublas_zgemm"])
PY
