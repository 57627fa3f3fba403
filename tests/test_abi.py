"""The C-ABI library loads on a CPU-only box and exports every symbol that
include/abft.h declares (no compute calls: there is no GPU here)."""
import os
import re

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _declared():
    src = open(os.path.join(ROOT, "include", "abft.h")).read()
    return re.findall(r"^ABFT_API\s+int\s+(\w+)\s*\(", src, flags=re.M)


def test_header_declares_the_hot_path():
    names = set(_declared())
    for n in ["abft_encode", "abft_verify", "abft_locate_correct", "abft_update_trsm", "abft_update_gemm",
              "abft_panel_potrf", "ft_potrf"]:
        assert n in names


def test_library_exports_every_declared_symbol():
    from paper_conf_sc_chenlllwtolzgc18_b200 import _lib

    lib = _lib.load()
    missing = [n for n in _declared() if not hasattr(lib, n)]
    assert not missing, missing


def test_binding_covers_every_declared_symbol():
    from paper_conf_sc_chenlllwtolzgc18_b200 import abft

    assert set(_declared()) <= set(abft.EXPORTS)


def test_host_only_entry_point():
    # abft_sizes is pure host arithmetic: 4/nb space overhead (L531) + 2/nb magnitudes
    from paper_conf_sc_chenlllwtolzgc18_b200 import abft

    c, r, cm, rm = abft.abft_sizes(30720, 30720, 512)
    assert c == r == 30720 * 30720 * 4 // 512 // 2 and cm == rm == c // 2
    assert (c + r) / 30720 ** 2 == 4 / 512


def test_illegal_arguments_rejected_without_gpu():
    from paper_conf_sc_chenlllwtolzgc18_b200 import abft

    lib = abft._L
    # null matrix pointer -> -1 (xerbla style); no device work is attempted
    assert lib.abft_encode(None, None, 3, None) == -1
    assert lib.abft_sizes(10, 10, 3, None, None, None, None) == -3


def test_host_lapack_for_the_host_pd_mode():
    # FT_PD_HOST (Alg. 2's CPU panel, L61) loads the OpenBLAS bundled with
    # SciPy; it must exist and export the LP64 symbols the library looks up
    import ctypes

    from paper_conf_sc_chenlllwtolzgc18_b200 import abft

    path = abft.host_lapack_path()
    lapack = ctypes.CDLL(path)
    for name in ("dpotrf_", "spotrf_", "dgetrf_", "sgetrf_", "dgeqrf_", "sgeqrf_"):
        assert hasattr(lapack, "scipy_" + name) or hasattr(lapack, name), name
    assert abft._L.ft_ctx_set_host_lapack(None, path.encode()) == -1
