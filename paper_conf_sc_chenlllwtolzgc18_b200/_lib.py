"""Locate and load libabft_b200.so (built in-tree by build.py).  Fails loudly:
there is no CPU fallback for any entry point."""
import ctypes
import os

HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(HERE, "libabft_b200.so")
_handle = None


def load():
    global _handle
    if _handle is None:
        if not os.path.exists(LIB_PATH):
            raise ImportError(
                f"{LIB_PATH} is missing: build it with `python -m paper_conf_sc_chenlllwtolzgc18_b200.build` "
                "(the CUDA path has no fallback)")
        _handle = ctypes.CDLL(LIB_PATH, mode=ctypes.RTLD_LOCAL)
    return _handle
