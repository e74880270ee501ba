"""Thin Python binding of include/granii.h (ctypes; argument marshalling only).

Every function has the ABI's name and forwards torch tensors as raw device
pointers plus the current CUDA stream.  All computation happens in
libgranii.so; there is no CPU fallback: if the library is missing this module
raises at import, and every compute call without a CUDA device returns
GRANII_ERR_CUDA, raised here as GraniiError.
"""
from __future__ import annotations

import ctypes
import os

import torch

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libgranii.so")

if not os.path.exists(LIB_PATH):
    raise ImportError(f"{LIB_PATH} is missing: run `python -c 'import __graft_entry__ as g; g.build()'` "
                      "(the CUDA library is required; there is no fallback)")
_lib = ctypes.CDLL(LIB_PATH)

# ---------------------------------------------------------------- constants (granii.h)
OK, ERR_INVALID_ARG, ERR_OOM, ERR_CUDA, ERR_NCCL, ERR_UNSUPPORTED, ERR_NOT_CALIBRATED = range(7)
ADD_SELF_LOOPS, SYMMETRIZE, BUILD_TRANSPOSE = 0x1, 0x2, 0x4
EPI_RELU = 0x1
SDDMM_DOT, SDDMM_ADD, SDDMM_LEAKYRELU, SDDMM_ROW_SOFTMAX = 0x0, 0x1, 0x10, 0x20
GEMM_TRANS_A, GEMM_TRANS_B, GEMM_RELU, GEMM_NO_STORE = 0x1, 0x2, 0x4, 0x8
GCN, GAT, SGC, TAGCN, GIN = 0, 1, 2, 3, 4
GCN_PRE_AGG, GCN_PRE_UPD, GCN_DYN_AGG, GCN_DYN_UPD = 0, 1, 2, 3
GAT_REUSE, GAT_RECOMP = 16, 17
GCN_COMPS = (GCN_PRE_AGG, GCN_PRE_UPD, GCN_DYN_AGG, GCN_DYN_UPD)
GAT_COMPS = (GAT_REUSE, GAT_RECOMP)
SGC_COMPS = (32, 33, 34, 35)
TAGCN_COMPS = (48, 49, 50, 51)
GIN_COMPS = (64, 65, 66, 67)
COMPS = {GCN: GCN_COMPS, GAT: GAT_COMPS, SGC: SGC_COMPS, TAGCN: TAGCN_COMPS, GIN: GIN_COMPS}
COMP_NAMES = {0: "GCN_PRE_AGG", 1: "GCN_PRE_UPD", 2: "GCN_DYN_AGG", 3: "GCN_DYN_UPD", 16: "GAT_REUSE",
              17: "GAT_RECOMP"}
for _m, _base in (("SGC", 32), ("TAGCN", 48), ("GIN", 64)):
    for _i, _v in enumerate(("PRE_AGG", "PRE_UPD", "DYN_AGG", "DYN_UPD")):
        COMP_NAMES[_base + _i] = f"{_m}_{_v}"
ACT_NONE, ACT_RELU = 0, 1
ATTN_ADDITIVE, ATTN_DOT = 0, 1
SELECT_NO_PREFILTER, SELECT_TRAINING, SELECT_INPUT_LAYER, SELECT_REFINE = 0x1, 0x2, 0x4, 0x8
MAX_CANDIDATES = 8
NUM_FEATURES = 8

_i64, _i32, _u32, _p, _f, _sz = (ctypes.c_int64, ctypes.c_int32, ctypes.c_uint32, ctypes.c_void_p,
                                 ctypes.c_float, ctypes.c_size_t)


class graph_info(ctypes.Structure):
    _fields_ = [("num_nodes", _i64), ("nnz", _i64), ("row_begin", _i64), ("row_end", _i64),
                ("local_nnz", _i64), ("max_local_rows", _i64), ("part_rank", _i32), ("part_world", _i32),
                ("symmetric", _i32), ("has_transpose", _i32), ("features", _i64 * NUM_FEATURES)]


class gemm_epilogue(ctypes.Structure):
    _fields_ = [("row_scale", _p), ("att_l", _p), ("att_r", _p), ("out_l", _p), ("out_r", _p)]


class layer_args(ctypes.Structure):
    _fields_ = [("K1", _i64), ("K2", _i64), ("H", _p), ("ldh", _i64), ("W", _p), ("a_l", _p), ("a_r", _p),
                ("act", _u32), ("attn", _u32), ("workspace", _p), ("workspace_bytes", _sz), ("comm", _p),
                ("d_a_l", _p), ("d_a_r", _p), ("hops", _i32), ("eps", _f), ("Kh", _i64), ("W2", _p)]


_SIGS = {
    "granii_last_error": ([], ctypes.c_char_p),
    "granii_version": ([], ctypes.c_char_p),
    "granii_graph_csr_create": ([_i64, _i64, _p, _p, _u32, _i32, _i32, _p, ctypes.POINTER(_p)], ctypes.c_int),
    "granii_graph_destroy": ([_p], ctypes.c_int),
    "granii_graph_query": ([_p, ctypes.POINTER(graph_info)], ctypes.c_int),
    "granii_graph_export_csr": ([_p, _p, _p], ctypes.c_int),
    "granii_graph_transpose_nnz": ([_p, ctypes.POINTER(_i64)], ctypes.c_int),
    "granii_graph_timings": ([_p, _p], ctypes.c_int),
    "granii_graph_export_transpose": ([_p, _p, _p], ctypes.c_int),
    "granii_graph_dinv": ([_p, ctypes.POINTER(_p)], ctypes.c_int),
    "granii_partition_bounds": ([_i64, _p, _i32, _p], ctypes.c_int),
    "granii_gather_layout_host": ([_i64, _p, _p, _i32, _i64, _p], ctypes.c_int),
    "granii_graph_export_local": ([_p, _p, _p], ctypes.c_int),
    "granii_spmm": ([_p, _p, _p, _i64, _i64, _p, _i64, _p, _p, _u32, _p], ctypes.c_int),
    "granii_sddmm": ([_p, _u32, _p, _i64, _p, _i64, _i64, _f, _p, _p], ctypes.c_int),
    "granii_gemm_workspace_size": ([_i64, _i64, _i64, _u32, ctypes.POINTER(_sz)], ctypes.c_int),
    "granii_gemm": ([_i64, _i64, _i64, _p, _i64, _p, _i64, _p, _i64, ctypes.POINTER(gemm_epilogue), _u32, _p, _sz,
                     _p], ctypes.c_int),
    "granii_layer_workspace_size": ([_p, ctypes.c_int, ctypes.c_int, _i64, _i64, ctypes.POINTER(_sz),
                                     ctypes.POINTER(_sz)], ctypes.c_int),
    "granii_layer_forward": ([_p, ctypes.c_int, ctypes.c_int, ctypes.POINTER(layer_args), _p, _i64, _p, _p],
                             ctypes.c_int),
    "granii_layer_backward": ([_p, ctypes.c_int, ctypes.c_int, ctypes.POINTER(layer_args), _p, _i64, _p, _i64, _p,
                               _p, _i64, _p, _p], ctypes.c_int),
    "granii_layer_workspace_size_ex": ([_p, ctypes.c_int, ctypes.c_int, ctypes.POINTER(layer_args),
                                        ctypes.POINTER(_sz), ctypes.POINTER(_sz)], ctypes.c_int),
    "granii_select_ex": ([_p, ctypes.c_int, ctypes.POINTER(layer_args), ctypes.c_char_p, _u32,
                          ctypes.POINTER(ctypes.c_int), ctypes.POINTER(_i32), ctypes.POINTER(ctypes.c_double),
                          ctypes.POINTER(_i32)], ctypes.c_int),
    "granii_select": ([_p, ctypes.c_int, _i64, _i64, ctypes.c_char_p, _u32, ctypes.POINTER(ctypes.c_int),
                       ctypes.POINTER(_i32), ctypes.POINTER(ctypes.c_double), ctypes.POINTER(_i32)], ctypes.c_int),
    "granii_cost_features": ([_p, _i32, _i64, _i64, ctypes.POINTER(ctypes.c_double), ctypes.POINTER(_i32),
                              ctypes.c_char_p], ctypes.c_int),
    "granii_comm_unique_id": ([_p], ctypes.c_int),
    "granii_comm_create": ([_p, _i32, _i32, ctypes.POINTER(_p)], ctypes.c_int),
    "granii_comm_destroy": ([_p], ctypes.c_int),
    "granii_comm_create_local": ([_i32, ctypes.POINTER(_p)], ctypes.c_int),
    "granii_comm_create_stub": ([_i32, _i32, ctypes.POINTER(_p)], ctypes.c_int),
    "granii_comm_stats": ([_p, ctypes.POINTER(ctypes.c_uint64), ctypes.POINTER(ctypes.c_uint64)], ctypes.c_int),
    "granii_comm_allgather": ([_p, _p, _p, _sz, _p], ctypes.c_int),
    "granii_comm_allreduce_sum": ([_p, _p, _sz, _p], ctypes.c_int),
    "granii_comm_query": ([_p, ctypes.POINTER(_i32), ctypes.POINTER(_i32), ctypes.POINTER(_i32)], ctypes.c_int),
    "granii_comm_plan": ([_p, _i64, _i32, _i32, ctypes.POINTER(_i32), ctypes.POINTER(ctypes.c_double),
                          ctypes.POINTER(ctypes.c_double)], ctypes.c_int),
    "granii_comm_watchdog": ([_p, _i64], ctypes.c_int),
    "granii_comm_check": ([_p], ctypes.c_int),
    "granii_comm_register": ([_p, _p, _sz, ctypes.POINTER(_p)], ctypes.c_int),
    "granii_comm_deregister": ([_p, _p], ctypes.c_int),
    "granii_debug_spin": ([_i64, _p], ctypes.c_int),
    "granii_softmax_xent": ([_i64, _i64, _p, _i64, _p, _i64, _p, _i64, _p, _p], ctypes.c_int),
    "granii_sgd": ([_i64, _f, _p, _p, _p], ctypes.c_int),
    "granii_profile_enable": ([_i32], ctypes.c_int),
    "granii_profile_read": ([_p, _i32, ctypes.POINTER(_i32)], ctypes.c_int),
    "granii_launch_count": ([], ctypes.c_int64),
}
for _name, (_args, _res) in _SIGS.items():
    _fn = getattr(_lib, _name)
    _fn.argtypes = _args
    _fn.restype = _res

EXPORTED = tuple(_SIGS)


class GraniiError(RuntimeError):
    def __init__(self, status: int, where: str):
        self.status = status
        super().__init__(f"{where}: status {status}: {_lib.granii_last_error().decode()}")


def _check(st: int, where: str):
    if st != OK:
        raise GraniiError(st, where)


def _ptr(t):
    if t is None:
        return None
    if isinstance(t, int):
        return t
    return t.data_ptr()


def _stream(stream=None):
    if stream is not None:
        return stream.cuda_stream if hasattr(stream, "cuda_stream") else stream
    return torch.cuda.current_stream().cuda_stream if torch.cuda.is_available() else None


def _ld(t):
    assert t.dim() == 2 and t.stride(1) == 1, "row-major 2-D tensor with unit column stride required"
    return t.stride(0)


def granii_version() -> str:
    return _lib.granii_version().decode()


def granii_last_error() -> str:
    return _lib.granii_last_error().decode()


# ---------------------------------------------------------------- graph
class Graph:
    """Owns a granii_graph handle (destroyed with the object)."""

    def __init__(self, handle: int):
        self.handle = handle
        self.info = granii_graph_query(handle)

    def __del__(self):
        if getattr(self, "handle", None) and _lib is not None:  # _lib is None at interpreter shutdown
            _lib.granii_graph_destroy(self.handle)
            self.handle = None

    @property
    def n_rows(self):
        return self.info.row_end - self.info.row_begin

    @property
    def nnz(self):
        return self.info.local_nnz

    def features(self):
        return list(self.info.features)


def granii_graph_csr_create(num_nodes: int, src: torch.Tensor, dst: torch.Tensor, flags: int = ADD_SELF_LOOPS,
                            part_rank: int = 0, part_world: int = 1, stream=None) -> Graph:
    assert src.dtype == torch.int32 and dst.dtype == torch.int32 and src.is_contiguous() and dst.is_contiguous()
    h = _p()
    _check(_lib.granii_graph_csr_create(num_nodes, src.numel(), _ptr(src), _ptr(dst), flags, part_rank, part_world,
                                        _stream(stream), ctypes.byref(h)), "granii_graph_csr_create")
    return Graph(h.value)


def granii_graph_query(handle) -> graph_info:
    info = graph_info()
    _check(_lib.granii_graph_query(handle, ctypes.byref(info)), "granii_graph_query")
    return info


def granii_graph_export_csr(g: Graph):
    import numpy as np
    rp = np.zeros(g.n_rows + 1, np.int64)
    ci = np.zeros(max(g.nnz, 1), np.int32)
    _check(_lib.granii_graph_export_csr(g.handle, rp.ctypes.data, ci.ctypes.data), "granii_graph_export_csr")
    return rp, ci[: g.nnz]


def granii_graph_timings(g: Graph) -> dict:
    """host ms of the creation phases"""
    ms = (ctypes.c_double * 4)()
    _check(_lib.granii_graph_timings(g.handle, ms), "granii_graph_timings")
    return {"csr_build": ms[0], "featurize": ms[1], "partition_schedule": ms[2], "transpose": ms[3]}


def granii_graph_export_transpose(g: Graph):
    """this rank's rows of Ãᵀ (BUILD_TRANSPOSE graphs): (row_ptr, global column ids)"""
    import numpy as np
    nt = _i64()
    _check(_lib.granii_graph_transpose_nnz(g.handle, ctypes.byref(nt)), "granii_graph_transpose_nnz")
    rp = np.zeros(g.n_rows + 1, np.int64)
    ci = np.zeros(max(nt.value, 1), np.int32)
    _check(_lib.granii_graph_export_transpose(g.handle, rp.ctypes.data, ci.ctypes.data),
           "granii_graph_export_transpose")
    return rp, ci[: nt.value]


def granii_graph_export_local(g: Graph):
    import numpy as np
    rp = np.zeros(g.n_rows + 1, np.int64)
    ci = np.zeros(max(g.nnz, 1), np.int32)
    _check(_lib.granii_graph_export_local(g.handle, rp.ctypes.data, ci.ctypes.data), "granii_graph_export_local")
    return rp, ci[: g.nnz]


def granii_gather_layout_host(cols, bounds, world: int, max_rows: int):
    import numpy as np
    c = np.ascontiguousarray(cols, dtype=np.int32)
    b = np.ascontiguousarray(bounds, dtype=np.int64)
    out = np.zeros(max(c.shape[0], 1), np.int32)
    _check(_lib.granii_gather_layout_host(c.shape[0], c.ctypes.data, b.ctypes.data, world, max_rows,
                                          out.ctypes.data), "granii_gather_layout_host")
    return out[: c.shape[0]]


def granii_graph_dinv(g: Graph) -> int:
    p = _p()
    _check(_lib.granii_graph_dinv(g.handle, ctypes.byref(p)), "granii_graph_dinv")
    return p.value


def granii_partition_bounds(row_ptr, world: int):
    import numpy as np
    rp = np.ascontiguousarray(row_ptr, dtype=np.int64)
    b = np.zeros(world + 1, np.int64)
    _check(_lib.granii_partition_bounds(rp.shape[0] - 1, rp.ctypes.data, world, b.ctypes.data),
           "granii_partition_bounds")
    return b


# ---------------------------------------------------------------- primitives
def granii_spmm(g: Graph, vals, X: torch.Tensor, K: int, Y: torch.Tensor, row_scale=None, col_scale=None,
                epilogue: int = 0, stream=None):
    _check(_lib.granii_spmm(g.handle, _ptr(vals), _ptr(X), _ld(X), K, _ptr(Y), _ld(Y), _ptr(row_scale),
                            _ptr(col_scale), epilogue, _stream(stream)), "granii_spmm")


def granii_sddmm(g: Graph, op: int, U, ldu: int, V, ldv: int, K: int, scale: float, out, stream=None):
    _check(_lib.granii_sddmm(g.handle, op, _ptr(U), ldu, _ptr(V), ldv, K, scale, _ptr(out), _stream(stream)),
           "granii_sddmm")


def granii_gemm_workspace_size(M: int, N: int, K: int, flags: int = 0) -> int:
    n = _sz()
    _check(_lib.granii_gemm_workspace_size(M, N, K, flags, ctypes.byref(n)), "granii_gemm_workspace_size")
    return n.value


def granii_gemm(M: int, N: int, K: int, A, lda: int, B, ldb: int, C, ldc: int, flags: int = 0, row_scale=None,
                att_l=None, att_r=None, out_l=None, out_r=None, workspace=None, stream=None):
    need = granii_gemm_workspace_size(M, N, K, flags)
    if workspace is None:
        workspace = torch.empty(max(need, 1), dtype=torch.uint8, device=A.device)
    ep = gemm_epilogue(_ptr(row_scale), _ptr(att_l), _ptr(att_r), _ptr(out_l), _ptr(out_r))
    _check(_lib.granii_gemm(M, N, K, _ptr(A), lda, _ptr(B), ldb, _ptr(C), ldc, ctypes.byref(ep), flags,
                            _ptr(workspace), workspace.numel(), _stream(stream)), "granii_gemm")


# ---------------------------------------------------------------- layers
def granii_layer_workspace_size(g: Graph, model: int, comp: int, K1: int, K2: int):
    ws, sv = _sz(), _sz()
    _check(_lib.granii_layer_workspace_size(g.handle, model, comp, K1, K2, ctypes.byref(ws), ctypes.byref(sv)),
           "granii_layer_workspace_size")
    return ws.value, sv.value


def make_layer_args(K1, K2, H, W, a_l=None, a_r=None, act=ACT_RELU, attn=ATTN_ADDITIVE, workspace=None,
                    comm=None, d_a_l=None, d_a_r=None, hops=0, eps=0.0, Kh=0, W2=None) -> layer_args:
    """d_a_l / d_a_r: GAT backward outputs (dL/da_l, dL/da_r), ignored by the forward.
    hops (SGC / TAGCN), eps / Kh / W2 (GIN): the other models' shape and weights."""
    return layer_args(K1, K2, _ptr(H), _ld(H) if H is not None else K1, _ptr(W), _ptr(a_l), _ptr(a_r), act, attn,
                      _ptr(workspace), workspace.numel() if workspace is not None else 0,
                      comm.handle if comm is not None else None, _ptr(d_a_l), _ptr(d_a_r), hops, eps, Kh, _ptr(W2))


def shape_args(K1, K2, hops=0, Kh=0) -> layer_args:
    """layer_args with only the shape fields set (sizing / selection)."""
    return layer_args(K1=K1, K2=K2, ldh=K1, hops=hops, Kh=Kh)


def granii_layer_workspace_size_ex(g: Graph, model: int, comp: int, args: layer_args):
    ws, sv = _sz(), _sz()
    _check(_lib.granii_layer_workspace_size_ex(g.handle, model, comp, ctypes.byref(args), ctypes.byref(ws),
                                               ctypes.byref(sv)), "granii_layer_workspace_size_ex")
    return ws.value, sv.value


def granii_select_ex(g: Graph, model: int, args: layer_args, calib_path: str | None = None, flags: int = 0):
    out = ctypes.c_int()
    cands = (_i32 * MAX_CANDIDATES)()
    pred = (ctypes.c_double * MAX_CANDIDATES)()
    n = _i32()
    _check(_lib.granii_select_ex(g.handle, model, ctypes.byref(args), calib_path.encode() if calib_path else None,
                                 flags, ctypes.byref(out), cands, pred, ctypes.byref(n)), "granii_select_ex")
    return out.value, {cands[i]: pred[i] for i in range(n.value)}


def granii_layer_forward(g: Graph, model: int, comp: int, args: layer_args, out: torch.Tensor, saved=None,
                         stream=None):
    _check(_lib.granii_layer_forward(g.handle, model, comp, ctypes.byref(args), _ptr(out), _ld(out), _ptr(saved),
                                     _stream(stream)), "granii_layer_forward")


def granii_layer_backward(g: Graph, model: int, comp: int, args: layer_args, out: torch.Tensor, dout: torch.Tensor,
                          saved, dH, dW: torch.Tensor, stream=None):
    _check(_lib.granii_layer_backward(g.handle, model, comp, ctypes.byref(args), _ptr(out), _ld(out), _ptr(dout),
                                      _ld(dout), _ptr(saved), _ptr(dH), _ld(dH) if dH is not None else 0, _ptr(dW),
                                      _stream(stream)), "granii_layer_backward")


def granii_select(g: Graph, model: int, K1: int, K2: int, calib_path: str | None = None, flags: int = 0):
    out = ctypes.c_int()
    cands = (_i32 * MAX_CANDIDATES)()
    pred = (ctypes.c_double * MAX_CANDIDATES)()
    n = _i32()
    _check(_lib.granii_select(g.handle, model, K1, K2, calib_path.encode() if calib_path else None, flags,
                              ctypes.byref(out), cands, pred, ctypes.byref(n)), "granii_select")
    return out.value, {cands[i]: pred[i] for i in range(n.value)}


P_SPMM_W, P_SPMM_U, P_SPMM_U_CS, P_SDDMM1, P_SDDMM1_SM, P_GEMM, P_GEMM_NOSTORE, P_GEMM_TN, P_ELEMENTWISE, \
    P_ALLGATHER, P_GEMM_ATT, P_GAT_BWD_A, P_GAT_BWD_B, P_GAT_DER = range(14)


def granii_cost_features(g: Graph, prim: int, K1: int, K2: int = 0):
    f = (ctypes.c_double * 16)()
    n = _i32()
    name = ctypes.create_string_buffer(32)
    _check(_lib.granii_cost_features(g.handle, prim, K1, K2, f, ctypes.byref(n), name), "granii_cost_features")
    return name.value.decode(), [f[i] for i in range(n.value)]


# ---------------------------------------------------------------- multi-GPU
class Comm:
    def __init__(self, handle: int, rank: int, world: int):
        self.handle, self.rank, self.world = handle, rank, world

    def __del__(self):
        if getattr(self, "handle", None):
            _lib.granii_comm_destroy(self.handle)
            self.handle = None


def granii_comm_unique_id() -> bytes:
    buf = ctypes.create_string_buffer(128)
    _check(_lib.granii_comm_unique_id(buf), "granii_comm_unique_id")
    return buf.raw


def granii_comm_create(uid: bytes, rank: int, world: int) -> Comm:
    buf = ctypes.create_string_buffer(uid, 128)
    h = _p()
    _check(_lib.granii_comm_create(buf, rank, world, ctypes.byref(h)), "granii_comm_create")
    return Comm(h.value, rank, world)


def granii_comm_allgather(c: Comm, send: torch.Tensor, recv: torch.Tensor, count: int, stream=None):
    _check(_lib.granii_comm_allgather(c.handle, _ptr(send), _ptr(recv), count, _stream(stream)),
           "granii_comm_allgather")


def granii_comm_allreduce_sum(c: Comm, buf: torch.Tensor, stream=None):
    _check(_lib.granii_comm_allreduce_sum(c.handle, _ptr(buf), buf.numel(), _stream(stream)),
           "granii_comm_allreduce_sum")


def granii_comm_query(c: Comm):
    """(nranks, rank, nccl_version) as the transport reports them"""
    n, r, v = _i32(), _i32(), _i32()
    _check(_lib.granii_comm_query(c.handle, ctypes.byref(n), ctypes.byref(r), ctypes.byref(v)), "granii_comm_query")
    return n.value, r.value, v.value


def granii_comm_plan(g: Graph, K: int, weighted: bool = False, col_scale: bool = False):
    """(phases, modelled ms of all-gather-then-SpMM, modelled ms of the planned schedule)"""
    P, a, b = _i32(), ctypes.c_double(), ctypes.c_double()
    _check(_lib.granii_comm_plan(g.handle, K, int(weighted), int(col_scale), ctypes.byref(P), ctypes.byref(a),
                                 ctypes.byref(b)), "granii_comm_plan")
    return P.value, a.value, b.value


def granii_comm_watchdog(c: Comm, timeout_ms: int):
    _check(_lib.granii_comm_watchdog(c.handle, int(timeout_ms)), "granii_comm_watchdog")


def granii_comm_check(c: Comm):
    _check(_lib.granii_comm_check(c.handle), "granii_comm_check")


def granii_comm_register(c: Comm, buf: torch.Tensor) -> int | None:
    h = _p()
    _check(_lib.granii_comm_register(c.handle, _ptr(buf), buf.numel() * buf.element_size(), ctypes.byref(h)),
           "granii_comm_register")
    return h.value


def granii_comm_deregister(c: Comm, handle):
    _check(_lib.granii_comm_deregister(c.handle, handle), "granii_comm_deregister")


def granii_debug_spin(us: int, stream=None):
    _check(_lib.granii_debug_spin(int(us), _stream(stream)), "granii_debug_spin")


def granii_comm_create_local(world: int) -> list:
    """In-process loopback group: one Comm per rank, each to be driven by its own
    thread (ctypes releases the GIL during the call) on its own stream of one GPU."""
    hs = (_p * world)()
    _check(_lib.granii_comm_create_local(world, hs), "granii_comm_create_local")
    return [Comm(hs[r], r, world) for r in range(world)]


def granii_comm_create_stub(rank: int, world: int) -> Comm:
    """TIMING STUB (collectives move no data): times one rank's local work on one GPU."""
    h = _p()
    _check(_lib.granii_comm_create_stub(rank, world, ctypes.byref(h)), "granii_comm_create_stub")
    return Comm(h.value, rank, world)


def granii_comm_stats(comm: Comm):
    """(bytes received by this rank, collective calls) since the communicator was created"""
    b, c = ctypes.c_uint64(), ctypes.c_uint64()
    _check(_lib.granii_comm_stats(comm.handle, ctypes.byref(b), ctypes.byref(c)), "granii_comm_stats")
    return b.value, c.value


# ---------------------------------------------------------------- training helpers
def granii_softmax_xent(Z: torch.Tensor, y: torch.Tensor, n_total: int, dZ: torch.Tensor, loss=None, stream=None):
    _check(_lib.granii_softmax_xent(Z.shape[0], Z.shape[1], _ptr(Z), _ld(Z), _ptr(y), n_total, _ptr(dZ), _ld(dZ),
                                    _ptr(loss), _stream(stream)), "granii_softmax_xent")


def granii_sgd(grad: torch.Tensor, param: torch.Tensor, lr: float, stream=None):
    _check(_lib.granii_sgd(param.numel(), lr, _ptr(grad), _ptr(param), _stream(stream)), "granii_sgd")


# ---------------------------------------------------------------- tracing
class prof_entry(ctypes.Structure):
    _fields_ = [("name", ctypes.c_char * 32), ("calls", _i64), ("launches", _i64), ("ms", ctypes.c_double),
                ("bytes", ctypes.c_double), ("flops", ctypes.c_double), ("compulsory_bytes", ctypes.c_double),
                ("l2_resident", _i64)]


def granii_profile_enable(on: bool = True):
    _check(_lib.granii_profile_enable(1 if on else 0), "granii_profile_enable")


def granii_profile_read() -> dict:
    arr = (prof_entry * 32)()
    n = _i32()
    _check(_lib.granii_profile_read(arr, 32, ctypes.byref(n)), "granii_profile_read")
    return {arr[i].name.decode(): {"calls": arr[i].calls, "launches": arr[i].launches, "ms": arr[i].ms,
                                   "bytes": arr[i].bytes, "flops": arr[i].flops,
                                   "compulsory_bytes": arr[i].compulsory_bytes, "l2_resident": arr[i].l2_resident}
            for i in range(n.value)}


def granii_launch_count() -> int:
    return int(_lib.granii_launch_count())
