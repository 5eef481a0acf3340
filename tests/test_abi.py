"""C-ABI boundary checks that need no GPU: the library loads, exports every
symbol include/bqr.h declares, validates arguments LAPACK-style without
touching memory, quick-returns, and reports its dispatch."""
import ctypes
import os
import re

import pytest

import paper_conf_ipps_andersonsk12_b200 as bqr

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "bqr.h")


@pytest.fixture(scope="module")
def lib():
    from paper_conf_ipps_andersonsk12_b200 import build
    build.build()
    return bqr.load()


def declared_symbols():
    txt = open(HEADER).read()
    txt = re.sub(r"/\*.*?\*/", "", txt, flags=re.S)
    return sorted(set(re.findall(r"\b(bqr_[a-z0-9_]+)\s*\(", txt)))


def test_header_declares_the_boundary():
    syms = declared_symbols()
    for s in ("bqr_geqrf_batched", "bqr_orgqr_batched", "bqr_apply_qh_batched", "bqr_status_string"):
        assert s in syms


def test_exports_every_declared_symbol(lib):
    for s in declared_symbols():
        assert hasattr(lib, s), s
        assert ctypes.cast(getattr(lib, s), ctypes.c_void_p).value


def test_version(lib):
    assert b"sm_100a" in lib.bqr_version()


FAKE = 0x1000  # never dereferenced: every call below returns before any launch


@pytest.mark.parametrize("args,code", [
    ((7, 4, 4, 1, FAKE, 4, FAKE), -1),          # bad dtype
    ((0, -1, 4, 1, FAKE, 4, FAKE), -2),
    ((0, 4, -1, 1, FAKE, 4, FAKE), -3),
    ((0, 4, 4, -1, FAKE, 4, FAKE), -4),
    ((0, 4, 4, 1, 0, 4, FAKE), -5),             # NULL A with work
    ((0, 4, 4, 1, FAKE, 3, FAKE), -6),          # lda < m
    ((0, 4, 4, 1, FAKE, 4, 0), -7),             # NULL tau
    ((0, 0, 4, 1, 0, 1, 0), 0),                 # quick return m == 0
    ((0, 4, 0, 1, 0, 4, 0), 0),                 # quick return n == 0
    ((1, 4, 4, 0, 0, 4, 0), 0),                 # quick return batch == 0
    ((0, 4, 4, 1, FAKE + 2, 4, FAKE), 3),       # misaligned fp32 pointer
    ((1, 4, 4, 1, FAKE + 4, 4, FAKE), 3),       # misaligned c64 pointer
    ((0, 3, 5, 1, FAKE, 3, FAKE), 1),           # m < n: not supported
    ((0, 4096, 4096, 1, FAKE, 4096, FAKE), 1),  # too large: not supported
])
def test_geqrf_argument_checks(lib, args, code):
    d, m, n, b, A, lda, tau = args
    st = lib.bqr_geqrf_batched(d, m, n, b, ctypes.c_void_p(A), lda, ctypes.c_void_p(tau), None)
    assert st == code


@pytest.mark.parametrize("args,code", [
    ((0, 4, 5, 4, 1, FAKE, 4, FAKE), -3),       # n > m
    ((0, 4, 4, 5, 1, FAKE, 4, FAKE), -4),       # k > n
    ((0, 4, 4, 4, -1, FAKE, 4, FAKE), -5),
    ((0, 4, 4, 4, 1, 0, 4, FAKE), -6),
    ((0, 4, 4, 4, 1, FAKE, 2, FAKE), -7),
    ((0, 4, 4, 4, 1, FAKE, 4, 0), -8),
    ((0, 4, 4, 4, 0, 0, 4, 0), 0),
])
def test_orgqr_argument_checks(lib, args, code):
    d, m, n, k, b, A, lda, tau = args
    assert lib.bqr_orgqr_batched(d, m, n, k, b, ctypes.c_void_p(A), lda, ctypes.c_void_p(tau), None) == code


@pytest.mark.parametrize("args,code", [
    ((0, 8, 4, 5, 1, 1, FAKE, 8, FAKE, FAKE, 8), -4),   # k > min(m,n)
    ((0, 8, 4, 4, -1, 1, FAKE, 8, FAKE, FAKE, 8), -5),
    ((0, 8, 4, 4, 1, -1, FAKE, 8, FAKE, FAKE, 8), -6),
    ((0, 8, 4, 4, 1, 1, FAKE, 7, FAKE, FAKE, 8), -8),
    ((0, 8, 4, 4, 1, 1, FAKE, 8, FAKE, 0, 8), -10),
    ((0, 8, 4, 4, 1, 1, FAKE, 8, FAKE, FAKE, 7), -11),
    ((0, 8, 4, 0, 1, 1, 0, 8, 0, FAKE, 8), 0),          # k == 0: nothing to do
    ((0, 8, 4, 4, 0, 1, 0, 8, 0, 0, 8), 0),             # nrhs == 0
])
def test_apply_argument_checks(lib, args, code):
    d, m, n, k, nrhs, b, A, lda, tau, B, ldb = args
    st = lib.bqr_apply_qh_batched(d, m, n, k, nrhs, b, ctypes.c_void_p(A), lda, ctypes.c_void_p(tau),
                                  ctypes.c_void_p(B), ldb, None)
    assert st == code


def test_status_strings(lib):
    for s in (-3, 0, 1, 2, 3, 99):
        assert lib.bqr_status_string(s)


@pytest.mark.parametrize("dt,m,n,expect", [
    (0, 4, 4, "tiny"), (0, 8, 8, "tiny"), (1, 8, 8, "tiny"),
    (0, 56, 56, "ll_f32_56x56_left4_x2"), (1, 240, 66, "rf_c64_R32G11_8x6_cta"),
    (0, 16, 16, "rf_f32"), (1, 100, 100, "rf_c64"), (0, 160, 160, "rf_f32_R16G16_10x10"),
    (0, 256, 256, "rf_f32_R32G32_8x8"), (0, 200, 64, "rf_f32_R32G8"), (1, 160, 160, "rf_c64_R16G32_10x5"), (1, 64, 64, "rf_c64_R8G8"), (0, 80, 80, "rf_f32_R8G8"),
])
def test_dispatch(lib, dt, m, n, expect):
    assert bqr.kernel_name(dt, m, n).startswith(expect)
    assert bqr.geqrf_launches(dt, m, n, 10) == 1


@pytest.mark.parametrize("dt,n,launches", [(1, 256, 17), (1, 192, 9), (1, 176, 9)])
def test_blocked_dispatch(lib, dt, n, launches):
    """Complex shapes above every single-SM class (c64 > 160: more words than
    one SM's register file) run the compact-WY blocked variant:
    per 96-column panel the register-file panel kernel, V extraction, four
    tensor-core GEMMs, xLARFT and the accumulate (8 launches) when trailing columns remain."""
    assert bqr.kernel_name(dt, n, n).startswith("wy_c64_panel96")
    assert bqr.geqrf_launches(dt, n, n, 10) == launches


@pytest.mark.parametrize("dt,n,launches", [(1, 255, 5), (1, 177, 3)])
def test_tiled_dispatch(lib, dt, n, launches):
    """Odd row counts (16-byte TMA rows impossible) keep the tiled panels:
    the register-file panel kernel + the Q^H B apply kernel per panel."""
    assert bqr.kernel_name(dt, n, n).startswith("tiled")
    assert bqr.geqrf_launches(dt, n, n, 10) == launches


def test_workspace_size(lib):
    w = bqr.host_workspace_bytes(0, 56, 56, 56, 100)
    assert w >= 2 * 100 * (56 * 56 + 56) * 4


def test_no_fallback_when_library_missing(monkeypatch, tmp_path):
    """The binding must fail loudly, never fall back to a CPU path."""
    import importlib
    mod = importlib.reload(bqr)
    monkeypatch.setattr(mod, "_LIB_PATH", str(tmp_path / "missing.so"))
    monkeypatch.setattr(mod, "_lib", None)
    with pytest.raises(mod.BQRError):
        mod.load()
    importlib.reload(bqr)


@pytest.mark.parametrize("args,code", [
    ((0, 8, 4, -1, 1, FAKE, 8, FAKE, FAKE, 8), -4),
    ((0, 8, 4, 1, 1, FAKE, 8, FAKE, 0, 8), -9),
    ((0, 8, 4, 1, 1, FAKE, 8, FAKE, FAKE, 7), -10),
    ((0, 8, 4, 1, 0, 0, 8, 0, 0, 8), 0),
])
def test_qhb_argument_checks(lib, args, code):
    d, m, n, nrhs, b, A, lda, tau, B, ldb = args
    st = lib.bqr_geqrf_qhb_batched(d, m, n, nrhs, b, ctypes.c_void_p(A), lda, ctypes.c_void_p(tau),
                                   ctypes.c_void_p(B), ldb, None)
    assert st == code


@pytest.mark.parametrize("args,code", [
    ((7, 8, 4, 1, 1, FAKE, 8, FAKE, FAKE, 8), -1),
    ((0, -1, 4, 1, 1, FAKE, 8, FAKE, FAKE, 8), -2),
    ((0, 8, -1, 1, 1, FAKE, 8, FAKE, FAKE, 8), -3),
    ((0, 8, 4, -1, 1, FAKE, 8, FAKE, FAKE, 8), -4),
    ((0, 8, 4, 1, -1, FAKE, 8, FAKE, FAKE, 8), -5),
    ((0, 8, 4, 1, 1, 0, 8, FAKE, FAKE, 8), -6),
    ((0, 8, 4, 1, 1, FAKE, 7, FAKE, FAKE, 8), -7),
    ((0, 8, 4, 1, 1, FAKE, 8, 0, FAKE, 8), -8),
    ((0, 8, 4, 1, 1, FAKE, 8, FAKE, 0, 8), -9),
    ((0, 8, 4, 1, 1, FAKE, 8, FAKE, FAKE, 7), -10),
    ((0, 8, 4, 1, 0, 0, 8, 0, 0, 8), 0),              # batch == 0: quick return
    ((0, 4, 8, 1, 1, FAKE, 4, FAKE, FAKE, 4), 1),     # m < n (minimum norm): not supported
    ((0, 8, 4, 1, 1, FAKE + 2, 8, FAKE, FAKE, 8), 3),  # misaligned
])
def test_gels_argument_checks(lib, args, code):
    d, m, n, nrhs, b, A, lda, tau, B, ldb = args
    st = lib.bqr_gels_batched(d, m, n, nrhs, b, ctypes.c_void_p(A), lda, ctypes.c_void_p(tau), ctypes.c_void_p(B),
                              ldb, None, None)
    assert st == code


# NEXT-3: LU without pivoting / Gauss-Jordan (argument checks run no kernel)
@pytest.mark.parametrize("args,code", [
    ((7, 8, 8, 1, FAKE, 8), -1),
    ((0, -1, 8, 1, FAKE, 8), -2),
    ((0, 8, -1, 1, FAKE, 8), -3),
    ((0, 8, 8, -1, FAKE, 8), -4),
    ((0, 8, 8, 1, 0, 8), -5),
    ((0, 8, 8, 1, FAKE, 7), -6),
    ((0, 8, 8, 0, 0, 8), 0),            # batch == 0: quick return
    ((0, 0, 8, 5, 0, 1), 0),            # m == 0: quick return
    ((0, 129, 129, 1, FAKE, 129), 1),   # beyond the size classes
    ((1, 8, 8, 1, FAKE + 4, 8), 3),     # complex pointer not 8-byte aligned
])
def test_getrf_np_argument_checks(lib, args, code):
    d, m, n, b, A, lda = args
    st = lib.bqr_getrf_np_batched(d, m, n, b, ctypes.c_void_p(A), lda, None, None)
    assert st == code


@pytest.mark.parametrize("args,code", [
    ((7, 8, 1, 1, FAKE, 8, FAKE, 8), -1),
    ((0, -1, 1, 1, FAKE, 8, FAKE, 8), -2),
    ((0, 8, -1, 1, FAKE, 8, FAKE, 8), -3),
    ((0, 8, 1, -1, FAKE, 8, FAKE, 8), -4),
    ((0, 8, 1, 1, 0, 8, FAKE, 8), -5),
    ((0, 8, 1, 1, FAKE, 7, FAKE, 8), -6),
    ((0, 8, 1, 1, FAKE, 8, 0, 8), -7),
    ((0, 8, 1, 1, FAKE, 8, FAKE, 7), -8),
    ((0, 8, 1, 0, 0, 8, 0, 8), 0),          # batch == 0
    ((0, 120, 9, 1, FAKE, 120, FAKE, 120), 1),  # n + nrhs > 128
    ((0, 8, 1, 1, FAKE + 2, 8, FAKE, 8), 3),
])
def test_gauss_jordan_argument_checks(lib, args, code):
    d, n, nrhs, b, A, lda, B, ldb = args
    st = lib.bqr_gauss_jordan_batched(d, n, nrhs, b, ctypes.c_void_p(A), lda, ctypes.c_void_p(B), ldb, None, None)
    assert st == code


def test_sass_proves_blackwell_native_instructions(lib):
    """libbqr.so is built for sm_100a and its SASS contains the instructions
    the design claims (B200_PROFILING.md "What proves a Blackwell-native
    kernel"): tcgen05 MMA (UTCHMMA, the compact-WY tensor-core GEMMs), TMA
    (UBLKCP bulk copies of the register-file kernels, UTMALDG in the GEMMs),
    packed FP32 (FFMA2), and no legacy HMMA."""
    import shutil
    import subprocess
    exe = shutil.which("cuobjdump") or "/usr/local/cuda/bin/cuobjdump"
    if not os.path.exists(exe):
        pytest.skip("cuobjdump not available")
    out = subprocess.run([exe, "-sass", bqr._LIB_PATH], capture_output=True, text=True, timeout=600).stdout
    assert "sm_100a" in subprocess.run([exe, "-lelf", bqr._LIB_PATH], capture_output=True, text=True).stdout
    for mnem in ("UTCHMMA", "UBLKCP", "UTMALDG", "FFMA2"):
        assert mnem in out, mnem
    assert " HMMA" not in out


def test_lu_kernel_names(lib):
    """bqr_lu_kernel_name mirrors the LU / Gauss-Jordan dispatch: the
    left-looking 56 x 56 fp32 LU, the register-file classes otherwise."""
    lib.bqr_lu_kernel_name.argtypes = [ctypes.c_int] * 5
    lib.bqr_lu_kernel_name.restype = ctypes.c_char_p
    assert lib.bqr_lu_kernel_name(0, 56, 56, 0, 0) == b"lll_f32_56x56_left4_x2"
    assert lib.bqr_lu_kernel_name(0, 56, 56, 1, 1) == b"llgj_f32_56x57_left4_x2"
    assert lib.bqr_lu_kernel_name(0, 56, 56, 2, 1) == b"lu_rf_R8G4_7x15_x2"
    assert lib.bqr_lu_kernel_name(1, 56, 56, 0, 0) == b"lu_rf_R16G8_4x8"
    assert lib.bqr_lu_kernel_name(0, 8, 8, 0, 0) == b"lu_rf_R4G4_2x2_x4"
    assert lib.bqr_lu_kernel_name(0, 129, 129, 0, 0) == b""


def test_left_looking_kernels_sass(lib):
    """The round-2 left-looking classes (C3 QR, L56 LU, GJ56 Gauss-Jordan):
    no divergence-guarded shuffles (BRA.DIV / WARPSYNC: their matrix loop
    runs on a shuffle-broadcast warp index), packed FP32 (FFMA2) in their
    updates, and at most 96 registers (17 warps = 34 matrices per SM; a
    scheduler holds 5 warps, 5 x 32 x 96 <= 16384)."""
    import re
    import shutil
    import subprocess
    exe = shutil.which("cuobjdump") or "/usr/local/cuda/bin/cuobjdump"
    if not os.path.exists(exe):
        pytest.skip("cuobjdump not available")
    names = {"_ZN3bqr2ll17geqrf_ll56_kernelENS0_6LlArgsE": "ll",
             "_ZN3bqr3lll18getrf_lll56_kernelENS0_4ArgsE": "lll",
             "_ZN3bqr4llgj16gj_llgj56_kernelENS0_4ArgsE": "llgj"}
    res = subprocess.run([exe, "-res-usage", bqr._LIB_PATH], capture_output=True, text=True, timeout=600).stdout
    for mangled in names:
        sass = subprocess.run([exe, "-sass", "-fun", mangled, bqr._LIB_PATH], capture_output=True, text=True,
                              timeout=600).stdout
        assert "FFMA2" in sass, mangled
        assert "BRA.DIV" not in sass and "WARPSYNC" not in sass, mangled
        m = re.search(re.escape(mangled) + r".*?\n\s*REG:(\d+)", res, re.S)
        assert m and int(m.group(1)) <= 96, (mangled, m and m.group(1))


def test_cluster_kernels_sass(lib):
    """The cluster-per-matrix classes (csrc/bqr_cl.cuh): the multi-CTA
    instantiations publish reflectors with st.async into distributed shared
    memory (SASS STAS) counted by mbarriers (SYNCS), with no GPU-scope fence
    on the per-column path (only the per-matrix cluster barrier's); the
    one-CTA instantiation uses plain shared stores; all use packed FP32
    (FFMA2) for the complex updates and spill nothing."""
    import re
    import shutil
    import subprocess
    exe = shutil.which("cuobjdump") or "/usr/local/cuda/bin/cuobjdump"
    if not os.path.exists(exe):
        pytest.skip("cuobjdump not available")
    res = subprocess.run([exe, "-res-usage", bqr._LIB_PATH], capture_output=True, text=True, timeout=600).stdout
    sass_all = subprocess.run([exe, "-sass", bqr._LIB_PATH], capture_output=True, text=True, timeout=600).stdout
    funcs = {}
    fn = None
    for line in sass_all.splitlines():
        m = re.search(r"Function : (\S+)", line)
        if m:
            fn = m.group(1)
            funcs.setdefault(fn, [])
        elif fn:
            funcs[fn].append(line)
    cl = {f: "\n".join(v) for f, v in funcs.items() if "geqrf_cl_kernel" in f}
    assert any("ILi4E" in f for f in cl) and any("ILi2E" in f for f in cl) and any("ILi1E" in f for f in cl), list(cl)
    for f, sass in cl.items():
        assert "FFMA2" in sass, f
        assert "SYNCS" in sass, f
        assert "LDL" not in sass and "STL" not in sass, f
        multi = "ILi1E" not in f.split("geqrf_cl_kernel")[1][:6]
        assert ("STAS" in sass) == multi, f
        assert sass.count("MEMBAR.ALL.GPU") <= 4, f  # the cluster barriers per matrix only
        m = re.search(re.escape(f) + r".*?\n\s*REG:\d+ STACK:(\d+)", res, re.S)
        assert m and int(m.group(1)) == 0, (f, m and m.group(1))
