"""Host-side checks of the C ABI (no GPU): the library builds for sm_100a, loads, and exports every
entry point include/lfd.h declares; the header and the binding agree; no product module imports the
oracle; the library refuses to run without a CUDA device (no CPU fallback)."""
import ctypes
import os
import re
import subprocess

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "lfd.h")


@pytest.fixture(scope="module")
def lib():
    from paper_conf_ipps_razakhllknvn24_b200 import build
    build.build()
    from paper_conf_ipps_razakhllknvn24_b200 import lfd
    return lfd.load()


def declared():
    txt = open(HEADER).read()
    return sorted(set(re.findall(r"^\s*(?:lfd_status|const char\*)\s+(lfd_\w+)\s*\(", txt, re.M)))


def test_header_declares_the_north_star_calls():
    d = declared()
    for name in ("lfd_init", "lfd_set_potential", "lfd_set_vector_potential", "lfd_step", "lfd_density_current"):
        assert name in d


def test_every_declared_symbol_is_exported(lib):
    from paper_conf_ipps_razakhllknvn24_b200 import lfd
    out = subprocess.run(["nm", "-D", "--defined-only", lfd.LIB_PATH], capture_output=True, text=True).stdout
    exported = set(re.findall(r" T (lfd_\w+)", out))
    for name in declared():
        assert name in exported, name
        assert hasattr(lib, name)
    assert set(declared()) == set(lfd.EXPORTS) | {"lfd_last_error"}


def test_library_is_sm100a_only(lib):
    from paper_conf_ipps_razakhllknvn24_b200 import lfd
    out = subprocess.run(["cuobjdump", "--list-elf", lfd.LIB_PATH], capture_output=True, text=True).stdout
    assert "sm_100a" in out
    sass = subprocess.run(["cuobjdump", "-sass", lfd.LIB_PATH], capture_output=True, text=True).stdout
    assert "DMMA" in sass  # FP64 tensor pipe in the projector GEMMs
    assert "UBLKCP" in sass  # TMA bulk copies staging the GEMM operands


def test_config_struct_layout_matches_header(lib):
    from paper_conf_ipps_razakhllknvn24_b200 import lfd
    # offsets fixed by the C struct in include/lfd.h (int32 x5, double x3, int32 x3, double, int32 x2)
    off = {f[0]: getattr(lfd.lfd_config, f[0]).offset for f in lfd.lfd_config._fields_}
    assert off["hx"] == 24 and off["bc"] == 48 and off["dt"] == 64 and off["flags"] == 76
    assert ctypes.sizeof(lfd.lfd_config) == 80


def test_no_cpu_fallback_without_device(lib):
    import torch
    if torch.cuda.is_available():
        pytest.skip("a GPU is present")
    from paper_conf_ipps_razakhllknvn24_b200 import lfd
    cfg = lfd.make_config(1, 4, 4, 4, 0.3, 0.3, 0.3, 0, 2, 0, 0.04)
    with pytest.raises(lfd.LFDError) as e:
        lfd.lfd_workspace_size(cfg)
    assert e.value.status == -3  # LFD_ECUDA


def test_validation_precedes_device_use(lib):
    from paper_conf_ipps_razakhllknvn24_b200 import lfd
    bad = lfd.make_config(1, 5, 4, 4, 0.3, 0.3, 0.3, 0, 2, 0, 0.04)  # odd n with periodic BC
    with pytest.raises(lfd.LFDError) as e:
        lfd.lfd_workspace_size(bad)
    assert e.value.status == -1 and "even" in str(e.value)
    bad = lfd.make_config(1, 4, 4, 4, 0.3, 0.3, 0.3, 0, 2, 0, 0.0)
    with pytest.raises(lfd.LFDError):
        lfd.lfd_workspace_size(bad)


def test_product_never_imports_oracle():
    pkg = os.path.join(ROOT, "paper_conf_ipps_razakhllknvn24_b200")
    for dirpath, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".cuh", ".h", ".cpp")):
                txt = open(os.path.join(dirpath, f)).read()
                assert "oracle" not in re.sub(r"(#|//).*", "", txt), f
