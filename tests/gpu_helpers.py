"""Shared helpers of the GPU parity tests: move seeded inputs to the device
in the C ABI's column-major layout and read results back for comparison with
the oracle.  Contains no method arithmetic."""
import numpy as np
import torch

from oracle import checksum as ck


def dev(A: np.ndarray, dtype=torch.float64, ld=None):
    from paper_conf_sc_chenlllwtolzgc18_b200 import abft

    t = torch.from_numpy(np.ascontiguousarray(A)).to(dtype)
    return abft.to_colmajor(t.cuda(), ld=ld)


def host(t: torch.Tensor) -> np.ndarray:
    return t.double().cpu().numpy()


def gpu_state_to_oracle(mat, prec="f64") -> ck.State:
    st = ck.State(A=host(mat.A), nb=mat.nb, prec=prec)
    st.colchk = host(mat.colchk)
    st.rowchk = host(mat.rowchk)
    st.colmag = None if mat.colmag is None else host(mat.colmag)
    st.rowmag = None if mat.rowmag is None else host(mat.rowmag)
    return st


def normwise_err(c_gpu, c_ref, X, axis):
    """Reading c-1: |c_gpu − c_ref| / Σ|X| (e) and / Σ(i+1)|X| (w)."""
    nb = X.shape[0]
    w = np.arange(1, nb + 1, dtype=np.float64)
    aX = np.abs(X)
    if axis == 0:  # column checksums, 2 x nb
        den_e = aX.sum(axis=0)
        den_w = w @ aX
        e = np.abs(c_gpu[0] - c_ref[0]) / np.maximum(den_e, 1e-300)
        ww = np.abs(c_gpu[1] - c_ref[1]) / np.maximum(den_w, 1e-300)
    else:  # row checksums, nb x 2
        den_e = aX.sum(axis=1)
        den_w = aX @ w
        e = np.abs(c_gpu[:, 0] - c_ref[:, 0]) / np.maximum(den_e, 1e-300)
        ww = np.abs(c_gpu[:, 1] - c_ref[:, 1]) / np.maximum(den_w, 1e-300)
    return max(float(e.max()), float(ww.max()))
