"""ctypes marshalling for oracle/granii_oracle.c (TEST INFRASTRUCTURE ONLY).

Arithmetic lives in the C file; this module only converts numpy/torch inputs to
contiguous fp64 / int arrays and back.  fp32 inputs are widened to fp64 exactly.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "granii_oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")

ADD_SELF_LOOPS = 0x1
SYMMETRIZE = 0x2
GCN_PRE_AGG, GCN_PRE_UPD, GCN_DYN_AGG, GCN_DYN_UPD = 0, 1, 2, 3
GAT_REUSE, GAT_RECOMP = 16, 17
GCN_COMPS = (GCN_PRE_AGG, GCN_PRE_UPD, GCN_DYN_AGG, GCN_DYN_UPD)
GAT_COMPS = (GAT_REUSE, GAT_RECOMP)
SGC_COMPS = (32, 33, 34, 35)      # PRE_AGG, PRE_UPD, DYN_AGG, DYN_UPD
TAGCN_COMPS = (48, 49, 50, 51)
GIN_COMPS = (64, 65, 66, 67)


def build(force: bool = False) -> str:
    """Compile liboracle.so with gcc (fp64, -O2, OpenMP over rows, no fast-math)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".{os.getpid()}.tmp"
        subprocess.check_call(["gcc", "-O2", "-fopenmp", "-fPIC", "-shared", "-std=c11",
                               "-fno-fast-math", _SRC, "-o", tmp, "-lm"])
        os.replace(tmp, _LIB)
    return _LIB


_lib = None


def lib():
    global _lib
    if _lib is None:
        _lib = ctypes.CDLL(build())
        i64, p = ctypes.c_int64, ctypes.c_void_p
        _lib.oracle_csr_build.argtypes = [i64, i64, p, p, ctypes.c_uint32, p, p, i64, p]
        _lib.oracle_partition.argtypes = [i64, p, i64, p]
        _lib.oracle_features.argtypes = [i64, p, p]
        _lib.oracle_dinv.argtypes = [i64, p, p]
        _lib.oracle_rowbcast.argtypes = [i64, i64, p, p, p]
        _lib.oracle_sddmm.argtypes = [i64, p, p, p, p, i64, p]
        _lib.oracle_spmm.argtypes = [i64, p, p, p, p, i64, p]
        _lib.oracle_spmm_t.argtypes = [i64, i64, p, p, p, p, i64, p]
        _lib.oracle_gemm.argtypes = [i64, i64, i64, p, ctypes.c_int, p, ctypes.c_int, p]
        _lib.oracle_gcn_forward.argtypes = [ctypes.c_int, i64, p, p, p, i64, p, i64, ctypes.c_int, p, p]
        _lib.oracle_gcn_rows.argtypes = [i64, p, p, p, p, p, i64, p, i64, ctypes.c_int, p]
        _lib.oracle_edge_softmax.argtypes = [i64, p, p, p]
        _lib.oracle_gat_rows.argtypes = [i64, p, p, p, p, i64, p, i64, p, p, ctypes.c_int, p]
        _lib.oracle_gat_forward.argtypes = [ctypes.c_int, ctypes.c_int, i64, p, p, p, i64, p, i64, p, p,
                                            ctypes.c_int, p, p]
        _lib.oracle_gat_backward.argtypes = [ctypes.c_int, i64, p, p, p, i64, p, i64, p, p, ctypes.c_int, p, p, p,
                                             p, p]
        _lib.oracle_gat_backward_magnitude.argtypes = _lib.oracle_gat_backward.argtypes
        _lib.oracle_sgc_forward.argtypes = [ctypes.c_int, i64, p, p, p, i64, p, i64, ctypes.c_int, ctypes.c_int, p]
        _lib.oracle_tagcn_forward.argtypes = [ctypes.c_int, i64, p, p, p, i64, p, i64, ctypes.c_int, ctypes.c_int, p]
        _lib.oracle_gin_forward.argtypes = [ctypes.c_int, i64, p, p, p, i64, p, i64, p, i64, ctypes.c_double,
                                            ctypes.c_int, p]
        _lib.oracle_gcn_backward.argtypes = [ctypes.c_int, i64, p, p, p, i64, p, i64, ctypes.c_int, p, p, p]
    return _lib


def _np(x, dtype):
    if hasattr(x, "detach"):
        x = x.detach().cpu().numpy()
    return np.ascontiguousarray(np.asarray(x), dtype=dtype)


def _p(a):
    return a.ctypes.data_as(ctypes.c_void_p) if a is not None else None


def csr_build(n, src, dst, flags=ADD_SELF_LOOPS):
    """O1: (row_ptr int64[N+1], col_idx int32[nnz]); raises ValueError on bad ids."""
    s, d = _np(src, np.int32), _np(dst, np.int32)
    E = s.shape[0]
    cap = E * (2 if flags & SYMMETRIZE else 1) + (n if flags & ADD_SELF_LOOPS else 0)
    rp = np.zeros(n + 1, np.int64)
    ci = np.zeros(max(cap, 1), np.int32)
    nnz = np.zeros(1, np.int64)
    rc = lib().oracle_csr_build(n, E, _p(s), _p(d), flags, _p(rp), _p(ci), cap, _p(nnz))
    if rc == 1:
        raise ValueError("edge id out of range")
    if rc != 0:
        raise MemoryError("oracle_csr_build failed")
    return rp, ci[: int(nnz[0])].copy()


def partition(row_ptr, G):
    rp = _np(row_ptr, np.int64)
    b = np.zeros(G + 1, np.int64)
    lib().oracle_partition(rp.shape[0] - 1, _p(rp), G, _p(b))
    return b


def features(row_ptr):
    rp = _np(row_ptr, np.int64)
    out = np.zeros(8, np.int64)
    lib().oracle_features(rp.shape[0] - 1, _p(rp), _p(out))
    return out


def dinv(row_ptr):
    rp = _np(row_ptr, np.int64)
    out = np.zeros(rp.shape[0] - 1, np.float64)
    lib().oracle_dinv(rp.shape[0] - 1, _p(rp), _p(out))
    return out


def rowbcast(d, B):
    d, B = _np(d, np.float64), _np(B, np.float64)
    C = np.zeros_like(B)
    lib().oracle_rowbcast(B.shape[0], B.shape[1], _p(d), _p(B), _p(C))
    return C


def sddmm(row_ptr, col_idx, U, V):
    rp, ci = _np(row_ptr, np.int64), _np(col_idx, np.int32)
    U, V = _np(U, np.float64), _np(V, np.float64)
    if U.ndim == 1:
        U, V = U[:, None].copy(), V[:, None].copy()
    out = np.zeros(ci.shape[0], np.float64)
    lib().oracle_sddmm(rp.shape[0] - 1, _p(rp), _p(ci), _p(U), _p(V), U.shape[1], _p(out))
    return out


def spmm(row_ptr, col_idx, vals, X):
    rp, ci = _np(row_ptr, np.int64), _np(col_idx, np.int32)
    X = _np(X, np.float64)
    v = _np(vals, np.float64) if vals is not None else None
    Y = np.zeros((rp.shape[0] - 1, X.shape[1]), np.float64)
    lib().oracle_spmm(rp.shape[0] - 1, _p(rp), _p(ci), _p(v), _p(X), X.shape[1], _p(Y))
    return Y


def spmm_t(row_ptr, col_idx, vals, X, n_cols):
    rp, ci = _np(row_ptr, np.int64), _np(col_idx, np.int32)
    X = _np(X, np.float64)
    v = _np(vals, np.float64) if vals is not None else None
    Y = np.zeros((n_cols, X.shape[1]), np.float64)
    lib().oracle_spmm_t(rp.shape[0] - 1, n_cols, _p(rp), _p(ci), _p(v), _p(X), X.shape[1], _p(Y))
    return Y


def gemm(A, B, ta=False, tb=False):
    A, B = _np(A, np.float64), _np(B, np.float64)
    M, K = (A.shape[1], A.shape[0]) if ta else A.shape
    N = B.shape[0] if tb else B.shape[1]
    C = np.zeros((M, N), np.float64)
    lib().oracle_gemm(M, N, K, _p(A), int(ta), _p(B), int(tb), _p(C))
    return C


def gcn_forward(comp, row_ptr, col_idx, H, W, act=1):
    """O3: returns (out, y_pre)."""
    rp, ci = _np(row_ptr, np.int64), _np(col_idx, np.int32)
    H, W = _np(H, np.float64), _np(W, np.float64)
    N, K1 = H.shape
    K2 = W.shape[1]
    y = np.zeros((N, K2), np.float64)
    o = np.zeros((N, K2), np.float64)
    rc = lib().oracle_gcn_forward(comp, N, _p(rp), _p(ci), _p(H), K1, _p(W), K2, act, _p(y), _p(o))
    if rc:
        raise ValueError(f"bad composition {comp}")
    return o, y


def gcn_rows(rows, row_ptr, col_idx, deg_of_col, H, W, act=1):
    rows = _np(rows, np.int64)
    rp, ci = _np(row_ptr, np.int64), _np(col_idx, np.int32)
    dg = _np(deg_of_col, np.int64)
    H, W = _np(H, np.float64), _np(W, np.float64)
    out = np.zeros((rows.shape[0], W.shape[1]), np.float64)
    lib().oracle_gcn_rows(rows.shape[0], _p(rows), _p(rp), _p(ci), _p(dg), _p(H), H.shape[1], _p(W),
                          W.shape[1], act, _p(out))
    return out


def gat_rows(rows, row_ptr, col_idx, H, W, a_l, a_r, act=0):
    """per-row definition of the (additive) GAT layer for sampled rows"""
    rows = _np(rows, np.int64)
    rp, ci = _np(row_ptr, np.int64), _np(col_idx, np.int32)
    H, W = _np(H, np.float64), _np(W, np.float64)
    al, ar = _np(a_l, np.float64), _np(a_r, np.float64)
    out = np.zeros((rows.shape[0], W.shape[1]), np.float64)
    lib().oracle_gat_rows(rows.shape[0], _p(rows), _p(rp), _p(ci), _p(H), H.shape[1], _p(W), W.shape[1], _p(al),
                          _p(ar), act, _p(out))
    return out


def edge_softmax(row_ptr, e):
    rp, e = _np(row_ptr, np.int64), _np(e, np.float64)
    a = np.zeros_like(e)
    lib().oracle_edge_softmax(rp.shape[0] - 1, _p(rp), _p(e), _p(a))
    return a


def gat_forward(comp, row_ptr, col_idx, H, W, a_l, a_r, act=0, dot=False):
    """O4: returns (out, alpha)."""
    rp, ci = _np(row_ptr, np.int64), _np(col_idx, np.int32)
    H, W = _np(H, np.float64), _np(W, np.float64)
    al, ar = _np(a_l, np.float64), _np(a_r, np.float64)
    N, K1 = H.shape
    K2 = W.shape[1]
    out = np.zeros((N, K2), np.float64)
    alpha = np.zeros(ci.shape[0], np.float64)
    rc = lib().oracle_gat_forward(comp, int(dot), N, _p(rp), _p(ci), _p(H), K1, _p(W), K2, _p(al), _p(ar),
                                  act, _p(out), _p(alpha))
    if rc:
        raise ValueError(f"bad composition {comp}")
    return out, alpha


def gcn_backward(comp, row_ptr, col_idx, H, W, G, act=1, need_dH=True):
    """O6: returns (dH or None, dW)."""
    rp, ci = _np(row_ptr, np.int64), _np(col_idx, np.int32)
    H, W, G = _np(H, np.float64), _np(W, np.float64), _np(G, np.float64)
    N, K1 = H.shape
    K2 = W.shape[1]
    dW = np.zeros((K1, K2), np.float64)
    dH = np.zeros((N, K1), np.float64) if need_dH else None
    rc = lib().oracle_gcn_backward(comp, N, _p(rp), _p(ci), _p(H), K1, _p(W), K2, act, _p(G), _p(dH), _p(dW))
    if rc:
        raise ValueError(f"bad composition {comp}")
    return dH, dW


def gat_backward(comp, row_ptr, col_idx, H, W, a_l, a_r, G, act=0, need_dH=True):
    """GAT backward (additive attention): returns (dH or None, dW, da_l, da_r)."""
    rp, ci = _np(row_ptr, np.int64), _np(col_idx, np.int32)
    H, W, G = _np(H, np.float64), _np(W, np.float64), _np(G, np.float64)
    al, ar = _np(a_l, np.float64), _np(a_r, np.float64)
    N, K1 = H.shape
    K2 = W.shape[1]
    dW = np.zeros((K1, K2), np.float64)
    dH = np.zeros((N, K1), np.float64) if need_dH else None
    dal = np.zeros(K2, np.float64)
    dar = np.zeros(K2, np.float64)
    rc = lib().oracle_gat_backward(comp, N, _p(rp), _p(ci), _p(H), K1, _p(W), K2, _p(al), _p(ar), act, _p(G),
                                   _p(dH), _p(dW), _p(dal), _p(dar))
    if rc:
        raise ValueError(f"bad composition {comp}")
    return dH, dW, dal, dar


def gat_backward_magnitude(comp, row_ptr, col_idx, H, W, a_l, a_r, G, act=0, need_dH=True):
    """Tolerance scale of the GAT backward (R19/R22): each gradient entry's sum of |terms|."""
    rp, ci = _np(row_ptr, np.int64), _np(col_idx, np.int32)
    H, W, G = _np(H, np.float64), _np(W, np.float64), _np(G, np.float64)
    al, ar = _np(a_l, np.float64), _np(a_r, np.float64)
    N, K1 = H.shape
    K2 = W.shape[1]
    dW = np.zeros((K1, K2), np.float64)
    dH = np.zeros((N, K1), np.float64) if need_dH else None
    dal = np.zeros(K2, np.float64)
    dar = np.zeros(K2, np.float64)
    rc = lib().oracle_gat_backward_magnitude(comp, N, _p(rp), _p(ci), _p(H), K1, _p(W), K2, _p(al), _p(ar), act,
                                             _p(G), _p(dH), _p(dW), _p(dal), _p(dar))
    if rc:
        raise ValueError(f"bad composition {comp}")
    return dH, dW, dal, dar


def sgc_forward(comp, row_ptr, col_idx, H, W, hops=2, act=0):
    """SGC (R23): sigma(S^k H W)."""
    rp, ci = _np(row_ptr, np.int64), _np(col_idx, np.int32)
    H, W = _np(H, np.float64), _np(W, np.float64)
    N, K1 = H.shape
    out = np.zeros((N, W.shape[1]), np.float64)
    if lib().oracle_sgc_forward(comp, N, _p(rp), _p(ci), _p(H), K1, _p(W), W.shape[1], hops, act, _p(out)):
        raise ValueError(f"bad composition {comp}")
    return out


def tagcn_forward(comp, row_ptr, col_idx, H, Ws, act=0):
    """TAGCN (R23): sigma(sum_j S^j H W_j); Ws has shape (hops+1, K1, K2)."""
    rp, ci = _np(row_ptr, np.int64), _np(col_idx, np.int32)
    H, Ws = _np(H, np.float64), _np(Ws, np.float64)
    N, K1 = H.shape
    hops, K2 = Ws.shape[0] - 1, Ws.shape[2]
    out = np.zeros((N, K2), np.float64)
    if lib().oracle_tagcn_forward(comp, N, _p(rp), _p(ci), _p(H), K1, _p(Ws), K2, hops, act, _p(out)):
        raise ValueError(f"bad composition {comp}")
    return out


def gin_forward(comp, row_ptr, col_idx, H, W1, W2, eps=0.0, act=0):
    """GIN (R23): sigma(ReLU(agg(H) W1) W2), agg = (1+eps) self + neighbour sum."""
    rp, ci = _np(row_ptr, np.int64), _np(col_idx, np.int32)
    H, W1, W2 = _np(H, np.float64), _np(W1, np.float64), _np(W2, np.float64)
    N, K1 = H.shape
    Kh, K2 = W1.shape[1], W2.shape[1]
    out = np.zeros((N, K2), np.float64)
    if lib().oracle_gin_forward(comp, N, _p(rp), _p(ci), _p(H), K1, _p(W1), Kh, _p(W2), K2, float(eps), act,
                                _p(out)):
        raise ValueError(f"bad composition {comp}")
    return out
