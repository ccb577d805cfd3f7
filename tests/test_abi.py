"""C-ABI checks that need no GPU (-m "not gpu").

* libblas3.so builds for sm_100a here and exports every symbol include/blas3.h
  declares;
* argument validation returns the reference-BLAS XERBLA position before any
  CUDA call (so it runs on a CPU-only box);
* quick returns (m=0, n=0, alpha=0&beta=1, ...) return 0 without touching
  the device;
* with no GPU a valid call reports BLAS3_ERR_CUDA instead of crashing.
"""
import ctypes
import os
import re
import subprocess

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HDR = os.path.join(ROOT, "include", "blas3.h")


@pytest.fixture(scope="module")
def lib():
    import __graft_entry__
    __graft_entry__.build()
    import paper_conf_ipps_cuiwxyf11_b200 as b
    return b


def declared_symbols():
    txt = open(HDR).read()
    txt = re.sub(r"/\*.*?\*/", "", txt, flags=re.S)
    return sorted(set(re.findall(r"\b(blas3_\w+)\s*\(", txt)))


def test_header_declares_the_six_routines():
    syms = declared_symbols()
    for r in ("sgemm", "ssymm", "ssyrk", "ssyr2k", "strmm", "strsm"):
        assert f"blas3_{r}" in syms


def test_all_declared_symbols_exported(lib):
    out = subprocess.run(["nm", "-D", "--defined-only", lib.LIB_PATH], capture_output=True,
                         text=True, check=True).stdout
    exported = set(re.findall(r"\b(blas3_\w+)\b", out))
    missing = [s for s in declared_symbols() if s not in exported]
    assert not missing, missing
    assert set(lib.EXPORTED) == set(declared_symbols())


def test_library_is_sm100a(lib):
    out = subprocess.run(["cuobjdump", "--list-elf", lib.LIB_PATH], capture_output=True, text=True).stdout
    assert "sm_100a" in out


NULL = None


def test_sgemm_xerbla(lib):
    f = lib.blas3_sgemm
    ok = dict(ta=b"N", tb=b"N", m=4, n=4, k=4, lda=4, ldb=4, ldc=4)

    def call(**kw):
        a = {**ok, **kw}
        return f(a["ta"], a["tb"], a["m"], a["n"], a["k"], 1.0, NULL, a["lda"], NULL, a["ldb"], 0.0,
                 NULL, a["ldc"], NULL)
    assert call(ta=b"X") == 1
    assert call(tb=b"Q") == 2
    assert call(m=-1) == 3
    assert call(n=-1) == 4
    assert call(k=-1) == 5
    assert call(lda=3) == 8
    assert call(ta=b"T", k=5, lda=4) == 8
    assert call(ldb=3) == 10
    assert call(tb=b"t", n=6, ldb=5) == 10
    assert call(ldc=3) == 13
    assert call(ta=b"X", m=-1) == 1              # first invalid argument wins
    # quick returns never touch the device or pointers
    assert call(m=0) == 0 and call(n=0) == 0
    assert f(b"N", b"N", 4, 4, 4, 0.0, NULL, 4, NULL, 4, 1.0, NULL, 4, NULL) == 0
    assert f(b"N", b"N", 4, 4, 0, 1.0, NULL, 4, NULL, 4, 1.0, NULL, 4, NULL) == 0
    assert call(ta=b"c") == 12                   # 'C' == 'T', lowercase accepted; then NULL C


def test_sgemm_streamed_xerbla(lib):
    f = lib.blas3_sgemm_streamed
    flag = (ctypes.c_uint32 * 4)()
    fp = ctypes.addressof(flag)
    ok = dict(ta=b"N", tb=b"N", m=4, n=4, k=64, lda=4, ldb=64, ldc=4, fl=fp, pk=32)

    def call(**kw):
        a = {**ok, **kw}
        return f(a["ta"], a["tb"], a["m"], a["n"], a["k"], 1.0, NULL, a["lda"], NULL, a["ldb"], 0.0,
                 NULL, a["ldc"], a["fl"], a["pk"], 1, NULL)
    assert call(ta=b"T") == 1                    # A's panels are K-ranges of its columns: 'N' only
    assert call(ta=b"X") == 1
    assert call(tb=b"Q") == 2
    assert call(m=-1) == 3 and call(n=-1) == 4 and call(k=-1) == 5
    assert call(lda=3) == 8 and call(ldb=63) == 10 and call(ldc=3) == 13
    assert call(fl=NULL) == 14
    assert call(pk=0) == 15 and call(pk=48) == 15 and call(pk=-32) == 15
    assert call(m=0) == 0                        # quick return before any device work
    assert lib.blas3_signal(NULL, 1, NULL) == 1
    assert lib.blas3_error_string(-5).decode().startswith("configuration not supported")


def test_ssymm_xerbla(lib):
    f = lib.blas3_ssymm
    call = lambda side=b"L", uplo=b"L", m=4, n=3, lda=4, ldb=4, ldc=4: f(  # noqa: E731
        side, uplo, m, n, 1.0, NULL, lda, NULL, ldb, 0.0, NULL, ldc, NULL)
    assert call(side=b"X") == 1
    assert call(uplo=b"X") == 2
    assert call(m=-2) == 3
    assert call(n=-2) == 4
    assert call(lda=3) == 7
    assert call(side=b"R", lda=2) == 7          # side=R: lda >= n = 3
    assert call(ldb=3) == 9
    assert call(ldc=3) == 12
    assert call(m=0) == 0


def test_ssyrk_ssyr2k_xerbla(lib):
    f = lib.blas3_ssyrk
    call = lambda uplo=b"U", tr=b"N", n=4, k=3, lda=4, ldc=4: f(uplo, tr, n, k, 1.0, NULL, lda, 0.0, NULL, ldc, NULL)  # noqa: E731
    assert call(uplo=b"Z") == 1
    assert call(tr=b"Z") == 2
    assert call(n=-1) == 3
    assert call(k=-1) == 4
    assert call(lda=3) == 7
    assert call(tr=b"T", lda=2) == 7             # trans=T: lda >= k = 3
    assert call(ldc=3) == 10
    assert call(n=0) == 0
    g = lib.blas3_ssyr2k
    call2 = lambda uplo=b"L", tr=b"T", n=4, k=3, lda=3, ldb=3, ldc=4: g(  # noqa: E731
        uplo, tr, n, k, 1.0, NULL, lda, NULL, ldb, 0.0, NULL, ldc, NULL)
    assert call2(uplo=b"x") == 1
    assert call2(tr=b"x") == 2
    assert call2(n=-1) == 3
    assert call2(k=-1) == 4
    assert call2(lda=2) == 7
    assert call2(ldb=2) == 9
    assert call2(ldc=3) == 12
    assert g(b"L", b"N", 4, 3, 0.0, NULL, 4, NULL, 4, 1.0, NULL, 4, NULL) == 0


@pytest.mark.parametrize("name", ["blas3_strmm", "blas3_strsm"])
def test_tr_xerbla(lib, name):
    f = getattr(lib, name)
    call = lambda s=b"L", u=b"U", t=b"N", d=b"N", m=4, n=5, lda=4, ldb=4: f(  # noqa: E731
        s, u, t, d, m, n, 1.0, NULL, lda, NULL, ldb, NULL)
    assert call(s=b"?") == 1
    assert call(u=b"?") == 2
    assert call(t=b"?") == 3
    assert call(d=b"?") == 4
    assert call(m=-1) == 5
    assert call(n=-1) == 6
    assert call(lda=3) == 9
    assert call(s=b"R", lda=4) == 9              # side=R: lda >= n = 5
    assert call(ldb=3) == 11
    assert call(m=0) == 0 and call(n=0) == 0
    assert call() == 10                          # B NULL but referenced


def test_no_gpu_reports_cuda_error_not_crash(lib):
    try:
        import torch
        if torch.cuda.is_available():
            pytest.skip("GPU present")
    except ImportError:
        pass
    buf = (ctypes.c_float * 16)()
    p = ctypes.addressof(buf)
    rc = lib.blas3_sgemm(b"N", b"N", 4, 4, 4, 1.0, p, 4, p, 4, 0.0, p, 4, NULL)
    assert rc < 0
    assert lib.blas3_error_string(rc)


def test_math_mode_and_misc(lib):
    old = lib.get_math_mode()
    assert lib.blas3_set_math_mode(7) == 1
    lib.set_math_mode("simt")
    assert lib.get_math_mode() == lib.MATH_SIMT_FP32
    lib.set_math_mode(old)
    assert lib.blas3_version() >= 100
    assert lib.blas3_error_string(-2).decode().startswith("current device")
    assert lib.blas3_error_string(5).decode().startswith("invalid argument")
    assert lib.launch_count() >= 0


def test_options_roundtrip_and_validation(lib):
    """Tuning options (blas3_set_option): defaults, valid updates, rejected
    values leave the option unchanged, unknown keys report INT64_MIN / 1."""
    assert lib.get_option("trsm_nb") in (128, 256, 512, 1024, 2048, 4096, 8192)
    with lib.options(trsm_nb=1024, gm_map=1, tc_cta=2):
        assert lib.get_option("trsm_nb") == 1024
        assert lib.get_option("gm_map") == 1
        assert lib.get_option("tc_cta") == 2
    assert lib.get_option("gm_map") in (-1, 0, 1)
    old = lib.get_option("trsm_nb")
    for bad in (100, 3000, 16384, -1):            # not a power of two in [128, 8192]
        assert lib.blas3_set_option(lib.OPTIONS["trsm_nb"], bad) == 1
    assert lib.get_option("trsm_nb") == old
    assert lib.blas3_set_option(lib.OPTIONS["tc_cta"], 3) == 1
    assert lib.blas3_set_option(99, 0) == 1
    assert lib.blas3_get_option(99) == -(2 ** 63)
    assert lib.get_option("tc_kc") == 3
    for bad in (0, -1, 65, 128):                  # in [1, 64]
        assert lib.blas3_set_option(lib.OPTIONS["tc_kc"], bad) == 1
    assert lib.get_option("tc_vec_store") == 1 and lib.get_option("tc_c_prefetch") == 1
    assert lib.get_option("max_sms") == 0
    assert lib.get_option("tc_c_async") == 0
    assert lib.get_option("trsm_panel") == 1
    assert len(lib.OPTIONS) == 27


def test_fp64_family_xerbla_and_quick_returns(lib):
    """The fp64 entry points share the s-routines' validators (csrc/validate.h):
    same XERBLA positions, same quick returns, all before any CUDA call."""
    g = lib.blas3_dgemm
    assert g(b"X", b"N", 4, 4, 4, 1.0, NULL, 4, NULL, 4, 0.0, NULL, 4, NULL) == 1
    assert g(b"N", b"N", 4, 4, 4, 1.0, NULL, 3, NULL, 4, 0.0, NULL, 4, NULL) == 8
    assert g(b"N", b"T", 4, 6, 4, 1.0, NULL, 4, NULL, 5, 0.0, NULL, 4, NULL) == 10
    assert g(b"N", b"N", 4, 4, 4, 1.0, NULL, 4, NULL, 4, 0.0, NULL, 3, NULL) == 13
    assert g(b"N", b"N", 0, 4, 4, 1.0, NULL, 4, NULL, 4, 0.0, NULL, 4, NULL) == 0
    assert g(b"N", b"N", 4, 4, 4, 0.0, NULL, 4, NULL, 4, 1.0, NULL, 4, NULL) == 0
    assert g(b"N", b"N", 4, 4, 4, 1.0, NULL, 4, NULL, 4, 0.0, NULL, 4, NULL) == 12   # NULL C
    s = lib.blas3_dsymm
    assert s(b"R", b"L", 4, 3, 1.0, NULL, 2, NULL, 4, 0.0, NULL, 4, NULL) == 7
    assert s(b"L", b"X", 4, 3, 1.0, NULL, 4, NULL, 4, 0.0, NULL, 4, NULL) == 2
    k = lib.blas3_dsyrk
    assert k(b"L", b"T", 5, 3, 1.0, NULL, 2, 0.0, NULL, 5, NULL) == 7
    assert k(b"L", b"N", 5, 3, 1.0, NULL, 5, 0.0, NULL, 4, NULL) == 10
    k2 = lib.blas3_dsyr2k
    assert k2(b"U", b"N", 5, 3, 1.0, NULL, 5, NULL, 4, 0.0, NULL, 5, NULL) == 9
    assert k2(b"U", b"N", 5, 3, 1.0, NULL, 5, NULL, 5, 0.0, NULL, 4, NULL) == 12
    for f in (lib.blas3_dtrmm, lib.blas3_dtrsm):
        assert f(b"L", b"L", b"N", b"X", 4, 4, 1.0, NULL, 4, NULL, 4, NULL) == 4
        assert f(b"R", b"L", b"N", b"N", 4, 6, 1.0, NULL, 5, NULL, 4, NULL) == 9
        assert f(b"L", b"L", b"N", b"N", 4, 6, 1.0, NULL, 4, NULL, 3, NULL) == 11
        assert f(b"L", b"L", b"N", b"N", 0, 6, 1.0, NULL, 1, NULL, 1, NULL) == 0
        assert f(b"L", b"L", b"N", b"N", 4, 6, 1.0, NULL, 4, NULL, 4, NULL) == 10     # NULL B


def test_fp64_wrappers_check_dtype_and_shape():
    """The tensor wrappers refuse fp32 tensors for d-routines (and the reverse)
    before any library call: marshalling only, no silent conversion."""
    torch = pytest.importorskip("torch")
    import paper_conf_ipps_cuiwxyf11_b200 as b
    a32 = torch.zeros((4, 4), dtype=torch.float32)
    a64 = torch.zeros((4, 4), dtype=torch.float64)
    with pytest.raises(TypeError):
        b.dgemm("N", "N", 1.0, a32, a32, 0.0, a32)
    with pytest.raises(TypeError):
        b.sgemm("N", "N", 1.0, a64, a64, 0.0, a64)
