"""C-ABI boundary checks that need no GPU (-m "not gpu").

* librgsqr.so builds for sm_100a, loads, and exports every function include/rgsqr.h declares;
* the Python binding binds exactly those names;
* host-side conventions (defaults, status strings, argument validation before any device
  work, RG_NO_DEVICE without a GPU) behave as documented.
"""
import ctypes
import os
import re
import subprocess

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "rgsqr.h")


@pytest.fixture(scope="module")
def rg():
    from paper_conf_hpdc_zhangbw20_b200 import _build
    _build.build()
    import paper_conf_hpdc_zhangbw20_b200 as rg
    return rg


def header_functions():
    txt = open(HEADER).read()
    return sorted(set(re.findall(r"RG_API\s+[\w\s\*]+?\b(\w+)\s*\(", txt)))


def test_header_declares_the_four_entry_points():
    fns = header_functions()
    for name in ("rgsqr_factor", "ls_solve_refined", "orthogonalize", "lowrank_approx"):
        assert name in fns


def test_library_exports_every_declared_symbol(rg):
    out = subprocess.check_output(["nm", "-D", "--defined-only", rg.LIB_PATH], text=True)
    exported = {ln.split()[-1] for ln in out.splitlines() if " T " in ln}
    missing = [f for f in header_functions() if f not in exported]
    assert not missing, missing
    # nothing else leaks out of the library (hidden visibility for internals)
    extra = sorted(s for s in exported if not s.startswith(("rg_", "rgsqr_", "orthogonalize", "ls_solve",
                                                             "lowrank_")))
    assert not extra, extra[:10]


def test_binding_covers_header(rg):
    assert sorted(rg.EXPORTS) == header_functions()
    L = rg.lib()
    for name in rg.EXPORTS:
        assert hasattr(L, name)


def test_library_is_sm100a(rg):
    out = subprocess.check_output(["cuobjdump", "--list-elf", rg.LIB_PATH], text=True)
    assert "sm_100a" in out
    sass = subprocess.check_output(["cuobjdump", "-sass", rg.LIB_PATH], text=True)
    assert "UTCHMMA" in sass          # tcgen05.mma
    assert "UTMALDG" in sass          # TMA tensor loads
    assert "LDTM" in sass             # tcgen05.ld (TMEM -> registers)
    # the recursive-update GEMMs (K1/K2 of every level above the leaf) are tcgen05 only; the only
    # mma.sync (HMMA) users are the leaf kernel's in-shared-memory 32-column K1/K2 (leaf.cu)
    funcs = sass.split("Function : ")
    hmma = sorted({f.split()[0] for f in funcs[1:] if " HMMA" in f})
    assert all("leaf_kernel" in name for name in hmma), hmma
    gemm = [f for f in funcs[1:] if "gemm_tc_kernel" in f.split()[0]]
    assert gemm and all(" HMMA" not in f for f in gemm)


def test_opts_defaults_and_status_strings(rg):
    o = rg.rg_opts()
    rg.lib().rg_opts_default(ctypes.byref(o))
    assert (o.precision, o.nb, o.scale, o.reortho, o.split, o.sync, o.panel) == (0, 32, 1, -1, 0, 1, 0)
    for code in range(8):
        assert rg.lib().rg_status_string(code)
    assert b"invalid" in rg.lib().rg_status_string(-3)
    assert rg.version().startswith("rgsqr")


def test_null_handle_is_argument_one(rg):
    L = rg.lib()
    o = rg.make_opts()
    assert L.rgsqr_factor(None, 10, 5, None, 10, None, 10, None, 5, ctypes.byref(o)) == -1
    assert L.orthogonalize(None, 10, 5, None, 10, None, 5, 1e-5, 2, None, None, ctypes.byref(o)) == -1
    assert L.ls_solve_refined(None, 10, 5, None, 10, None, None, 1e-10, 10, None, None, ctypes.byref(o)) == -1
    assert L.lowrank_approx(None, 10, 5, None, 10, 2, 1, 1, 0, None, 10, None, None, 5, ctypes.byref(o)) == -1


def test_create_without_gpu_reports_no_device(rg):
    import torch
    if torch.cuda.is_available():
        pytest.skip("GPU present")
    h = ctypes.c_void_p()
    st = rg.lib().rg_create(ctypes.byref(h), 0, None)
    assert st == rg.RG_NO_DEVICE
    with pytest.raises(rg.RGError):
        rg.Handle(0, stream=0)


def test_nccl_unique_id_without_gpu(rg):
    path = rg._find_nccl()
    if not path:
        pytest.skip("no libnccl")
    assert rg.lib().rg_nccl_load(path.encode()) == rg.RG_OK
    buf = (ctypes.c_char * 128)()
    assert rg.lib().rg_comm_unique_id(buf) == rg.RG_OK
    assert any(b != 0 for b in bytearray(buf.raw))
