"""Pins of the fp64 oracle against things other than itself (-m "not gpu").

Each pin is chosen so a plausible mistake (dropped term, wrong sign/index,
transposed operand, wrong degree, missing self-loop, wrong softmax axis) fails:
  * brute-force dense matrices built straight from the raw edge list with set
    semantics (no CSR code involved) -- PAPER.md Eq. 2 (L115), Eq. 3 (L123);
  * closed forms (identity graph, complete graph, k-regular graph, W = I,
    zero attention weights, self-loop-only GAT);
  * the paper's own association example A_d·B_s·C_d·D_d (L41);
  * a hand-derived worked example (tests/golden/hypercube_q3.json);
  * central finite differences for the backward pass;
  * numpy library routines (matmul, sort) where the step is one.
"""
import json
import os

import numpy as np
import pytest

import oracle as O
from paper_conf_cgo_lenadorasgytm26_b200 import synth

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def dense_adj(n, src, dst, sym, loops):
    """Ã from the raw edge list: A[dst, src] = 1 (messages src -> dst, L192)."""
    A = np.zeros((n, n))
    s, d = np.asarray(src), np.asarray(dst)
    A[d, s] = 1.0
    if sym:
        A[s, d] = 1.0
    if loops:
        A[np.arange(n), np.arange(n)] = 1.0
    return A


def rel(a, b):
    return np.max(np.abs(a - b)) / max(np.max(np.abs(b)), 1e-300)


def small_graph(seed, n=23, m=60):
    s, d = synth.random_small(n, m, seed)
    return n, s.numpy(), d.numpy()


FLAGS = [0, O.ADD_SELF_LOOPS, O.SYMMETRIZE, O.ADD_SELF_LOOPS | O.SYMMETRIZE]


# ------------------------------------------------------------------ O1 / O2 / O8
@pytest.mark.parametrize("flags", FLAGS)
@pytest.mark.parametrize("seed", [0, 1, 2])
def test_csr_matches_dense_pattern(flags, seed):
    n, s, d = small_graph(seed)
    rp, ci = O.csr_build(n, s, d, flags)
    A = dense_adj(n, s, d, flags & O.SYMMETRIZE, flags & O.ADD_SELF_LOOPS)
    assert rp[0] == 0 and rp[-1] == ci.shape[0] == int(A.sum())
    assert np.all(np.diff(rp) >= 0)
    for r in range(n):
        cols = ci[rp[r]:rp[r + 1]]
        assert np.all(np.diff(cols) > 0), "columns strictly increasing"
        assert np.array_equal(cols, np.nonzero(A[r])[0])


def test_csr_symmetric_equals_transpose_and_edge_cases():
    n, s, d = small_graph(7)
    rp, ci = O.csr_build(n, s, d, O.SYMMETRIZE | O.ADD_SELF_LOOPS)
    A = np.zeros((n, n))
    for r in range(n):
        A[r, ci[rp[r]:rp[r + 1]]] = 1
    assert np.array_equal(A, A.T)
    assert np.all(np.diag(A) == 1)
    rp0, ci0 = O.csr_build(5, np.zeros(0, np.int32), np.zeros(0, np.int32), O.ADD_SELF_LOOPS)
    assert list(rp0) == [0, 1, 2, 3, 4, 5] and list(ci0) == [0, 1, 2, 3, 4]
    rp1, ci1 = O.csr_build(5, np.zeros(0, np.int32), np.zeros(0, np.int32), 0)
    assert list(rp1) == [0] * 6 and ci1.shape[0] == 0
    with pytest.raises(ValueError):
        O.csr_build(5, np.array([0, 5], np.int32), np.array([1, 1], np.int32), 0)
    with pytest.raises(ValueError):
        O.csr_build(5, np.array([0, -1], np.int32), np.array([1, 1], np.int32), 0)


@pytest.mark.parametrize("G", [1, 2, 3, 4, 8, 40])
def test_partition_owns_every_row_once(G):
    n, s, d = small_graph(3, n=31, m=120)
    rp, _ = O.csr_build(n, s, d, O.SYMMETRIZE | O.ADD_SELF_LOOPS)
    b = O.partition(rp, G)
    assert b[0] == 0 and b[-1] == n and np.all(np.diff(b) >= 0)
    nnz = rp[-1]
    for g in range(1, G):
        target = -(-g * nnz // G)
        assert b[g] == np.searchsorted(rp, target, side="left")   # library lower_bound
    owned = np.concatenate([np.arange(b[g], b[g + 1]) for g in range(G)])
    assert np.array_equal(owned, np.arange(n))


def test_features_match_numpy():
    n, s, d = small_graph(4, n=250, m=900)
    rp, _ = O.csr_build(n, s, d, O.SYMMETRIZE)
    f = O.features(rp)
    deg = np.diff(rp)
    k = -(-n // 100)
    assert list(f) == [n, rp[-1], deg.sum(), (deg * deg).sum(), deg.max(), deg.min(),
                       np.sort(deg)[::-1][:k].sum(), (deg == 0).sum()]


def test_dinv_definition():
    rp = np.array([0, 1, 1, 5, 9, 18], np.int64)    # degrees 1, 0, 4, 4, 9
    assert np.array_equal(O.dinv(rp), np.array([1.0, 0.0, 0.5, 0.5, 1.0 / 3.0]))


# ------------------------------------------------------------------ O5 primitives
def csr_and_dense(seed, n=29, m=140, flags=O.SYMMETRIZE | O.ADD_SELF_LOOPS):
    s, d = synth.random_small(n, m, seed)
    rp, ci = O.csr_build(n, s, d, flags)
    A = dense_adj(n, s.numpy(), d.numpy(), flags & O.SYMMETRIZE, flags & O.ADD_SELF_LOOPS)
    return rp, ci, A


def test_sddmm_is_masked_dense_product():
    rp, ci, A = csr_and_dense(11, flags=O.ADD_SELF_LOOPS)   # directed: U and V roles must not swap
    rng = np.random.default_rng(0)
    U, V = rng.standard_normal((29, 7)), rng.standard_normal((29, 7))
    out = O.sddmm(rp, ci, U, V)
    P = U @ V.T
    rows = np.repeat(np.arange(29), np.diff(rp))
    assert rel(out, P[rows, ci]) < 1e-13


@pytest.mark.parametrize("weighted", [False, True])
def test_spmm_and_transpose_are_dense_products(weighted):
    rp, ci, A = csr_and_dense(12, flags=O.ADD_SELF_LOOPS)
    rng = np.random.default_rng(1)
    X = rng.standard_normal((29, 5))
    vals = rng.standard_normal(ci.shape[0]) if weighted else None
    S = A.copy()
    if weighted:
        rows = np.repeat(np.arange(29), np.diff(rp))
        S[rows, ci] = vals
    assert rel(O.spmm(rp, ci, vals, X), S @ X) < 1e-13
    assert rel(O.spmm_t(rp, ci, vals, X, 29), S.T @ X) < 1e-13


@pytest.mark.parametrize("ta,tb", [(0, 0), (1, 0), (0, 1), (1, 1)])
def test_gemm_is_library_matmul(ta, tb):
    rng = np.random.default_rng(2)
    A = rng.standard_normal((13, 9) if not ta else (9, 13))
    B = rng.standard_normal((9, 6) if not tb else (6, 9))
    ref = (A.T if ta else A) @ (B.T if tb else B)
    assert rel(O.gemm(A, B, ta, tb), ref) < 1e-13


def test_rowbcast_eq1():
    d = np.array([2.0, -1.0, 0.5])
    B = np.arange(6.0).reshape(3, 2)
    assert np.array_equal(O.rowbcast(d, B), np.array([[0, 2], [-2, -3], [2, 2.5]]))


# ------------------------------------------------------------------ O3 GCN forward
def dense_gcn(A, H, W, act):
    deg = A.sum(1)
    dm = np.where(deg > 0, 1.0 / np.sqrt(np.where(deg > 0, deg, 1)), 0.0)
    Y = np.diag(dm) @ A @ np.diag(dm) @ H @ W
    return np.maximum(Y, 0) if act else Y, Y


@pytest.mark.parametrize("comp", O.GCN_COMPS)
@pytest.mark.parametrize("flags", [O.SYMMETRIZE | O.ADD_SELF_LOOPS, O.ADD_SELF_LOOPS, O.SYMMETRIZE])
def test_gcn_compositions_equal_dense_definition(comp, flags):
    rp, ci, A = csr_and_dense(21, n=37, m=150, flags=flags)
    rng = np.random.default_rng(3)
    H, W = rng.uniform(-1, 1, (37, 9)), rng.uniform(-1, 1, (9, 5))
    for act in (0, 1):
        out, y = O.gcn_forward(comp, rp, ci, H, W, act)
        ref_out, ref_y = dense_gcn(A, H, W, act)
        assert rel(y, ref_y) < 1e-12
        assert rel(out, ref_out) < 1e-12


def test_gcn_compositions_agree_with_each_other():
    rp, ci, _ = csr_and_dense(22, n=200, m=900)
    rng = np.random.default_rng(4)
    H, W = rng.uniform(-1, 1, (200, 24)), rng.uniform(-1, 1, (24, 40))
    outs = [O.gcn_forward(c, rp, ci, H, W, 1)[1] for c in O.GCN_COMPS]
    for o in outs[1:]:
        assert rel(o, outs[0]) < 1e-12


def test_gcn_identity_graph_is_plain_matmul():
    n = 17
    rp, ci = O.csr_build(n, np.zeros(0, np.int32), np.zeros(0, np.int32), O.ADD_SELF_LOOPS)
    rng = np.random.default_rng(5)
    H, W = rng.standard_normal((n, 6)), rng.standard_normal((6, 4))
    for comp in O.GCN_COMPS:
        _, y = O.gcn_forward(comp, rp, ci, H, W, 0)
        assert rel(y, H @ W) < 1e-14


def test_gcn_complete_graph_is_column_mean():
    n = 9
    s, d = synth.complete(n)
    rp, ci = O.csr_build(n, s, d, O.SYMMETRIZE | O.ADD_SELF_LOOPS)
    rng = np.random.default_rng(6)
    H, W = rng.standard_normal((n, 5)), rng.standard_normal((5, 3))
    ref = np.tile((H @ W).mean(0), (n, 1))          # M = J / n
    for comp in O.GCN_COMPS:
        assert rel(O.gcn_forward(comp, rp, ci, H, W, 0)[1], ref) < 1e-13


def test_gcn_regular_graph_constant_rows():
    n, k = 20, 4
    s, d = synth.ring(n, k)
    rp, ci = O.csr_build(n, s, d, O.SYMMETRIZE | O.ADD_SELF_LOOPS)
    assert np.all(np.diff(rp) == k + 1)
    h = np.array([0.5, -2.0, 1.25])
    H = np.tile(h, (n, 1))
    W = np.array([[1.0, 2.0], [0.0, -1.0], [3.0, 0.5]])
    for comp in O.GCN_COMPS:
        assert rel(O.gcn_forward(comp, rp, ci, H, W, 0)[1], np.tile(h @ W, (n, 1))) < 1e-14
    # W = I: the layer is the normalised SpMM, M = Ã / (k+1)
    rng = np.random.default_rng(8)
    X = rng.standard_normal((n, 3))
    A = dense_adj(n, s.numpy(), d.numpy(), True, True)
    assert rel(O.gcn_forward(0, rp, ci, X, np.eye(3), 0)[1], A @ X / (k + 1)) < 1e-14


def test_gcn_golden_hypercube():
    """Hand-derived worked example (tests/golden/hypercube_q3.json)."""
    g = json.load(open(os.path.join(GOLDEN, "hypercube_q3.json")))
    n = 8
    src = [i for i in range(n) for b in range(3) if i < (i ^ (1 << b))]
    dst = [i ^ (1 << b) for i in range(n) for b in range(3) if i < (i ^ (1 << b))]
    rp, ci = O.csr_build(n, np.array(src, np.int32), np.array(dst, np.int32), O.SYMMETRIZE | O.ADD_SELF_LOOPS)
    H = np.array(g["H"], float)
    W = np.array(g["W"], float)
    for comp in O.GCN_COMPS:
        out, y = O.gcn_forward(comp, rp, ci, H, W, 1)
        assert np.allclose(y, np.array(g["Y"]), rtol=0, atol=1e-14)


def test_paper_l41_association_example():
    """L41: ((A_d·B_s·C_d)·D_d) = {SDDMM, SpMM} equals (A_d·(B_s·(C_d·D_d))) = {GEMM, SpMM, GEMM}."""
    rp, ci, A = csr_and_dense(31, n=26, m=90)
    d = O.dinv(rp)
    rng = np.random.default_rng(9)
    Dd = rng.standard_normal((26, 4))
    nval = O.sddmm(rp, ci, d, d)                                   # (A_d · B_s · C_d) by SDDMM
    left = O.spmm(rp, ci, nval, Dd)                                # (...) · D_d by SpMM
    right = O.gemm(np.diag(d), O.spmm(rp, ci, None, O.gemm(np.diag(d), Dd)))
    assert rel(left, right) < 1e-13
    assert rel(left, np.diag(d) @ A @ np.diag(d) @ Dd) < 1e-13


def test_gcn_rows_matches_full_forward():
    rp, ci, _ = csr_and_dense(41, n=120, m=500)
    rng = np.random.default_rng(10)
    H, W = rng.uniform(-1, 1, (120, 11)), rng.uniform(-1, 1, (11, 7))
    full = O.gcn_forward(1, rp, ci, H, W, 1)[0]
    rows = np.array([0, 5, 17, 119, 64])
    sub = O.gcn_rows(rows, rp, ci, np.diff(rp), H, W, 1)
    assert rel(sub, full[rows]) < 1e-13


# ------------------------------------------------------------------ O4 GAT forward
def dense_gat(A, H, W, al, ar, dot, comp):
    T = H @ W
    if dot:
        S = (T @ T.T) / np.sqrt(W.shape[1])
    else:
        S = (T @ al)[:, None] + (T @ ar)[None, :]
        S = np.where(S > 0, S, 0.2 * S)
    S = np.where(A > 0, S, -np.inf)
    m = S.max(1, keepdims=True)
    P = np.where(A > 0, np.exp(S - m), 0.0)
    alpha = P / P.sum(1, keepdims=True)
    return (alpha @ T) if comp == O.GAT_REUSE else (alpha @ H) @ W, alpha


@pytest.mark.parametrize("comp", O.GAT_COMPS)
@pytest.mark.parametrize("dot", [False, True])
def test_gat_matches_dense_masked_softmax(comp, dot):
    rp, ci, A = csr_and_dense(51, n=33, m=160, flags=O.ADD_SELF_LOOPS)   # directed
    rng = np.random.default_rng(11)
    H, W = rng.uniform(-1, 1, (33, 6)), rng.uniform(-1, 1, (6, 10))
    al, ar = rng.uniform(-1, 1, 10), rng.uniform(-1, 1, 10)
    out, alpha = O.gat_forward(comp, rp, ci, H, W, al, ar, 0, dot)
    ref, ref_alpha = dense_gat(A, H, W, al, ar, dot, comp)
    rows = np.repeat(np.arange(33), np.diff(rp))
    assert rel(out, ref) < 1e-12
    assert rel(alpha, ref_alpha[rows, ci]) < 1e-12
    sums = np.add.reduceat(alpha, rp[:-1])
    assert np.allclose(sums, 1.0, atol=1e-14)


def test_gat_rows_matches_dense_definition():
    rp, ci, A = csr_and_dense(54, n=40, m=200, flags=O.ADD_SELF_LOOPS)
    rng = np.random.default_rng(16)
    H, W = rng.uniform(-1, 1, (40, 5)), rng.uniform(-1, 1, (5, 9))
    al, ar = rng.uniform(-1, 1, 9), rng.uniform(-1, 1, 9)
    ref, _ = dense_gat(A, H, W, al, ar, False, O.GAT_REUSE)
    rows = np.array([0, 3, 17, 39, 22])
    assert rel(O.gat_rows(rows, rp, ci, H, W, al, ar), ref[rows]) < 1e-12
    assert rel(O.gat_rows(rows, rp, ci, H, W, al, ar, act=1), np.maximum(ref[rows], 0)) < 1e-12


def test_gat_closed_forms():
    rp, ci, A = csr_and_dense(52, n=25, m=100)
    rng = np.random.default_rng(12)
    H, W = rng.uniform(-1, 1, (25, 4)), rng.uniform(-1, 1, (4, 8))
    z = np.zeros(8)
    for comp in O.GAT_COMPS:       # zero attention weights: alpha = D^-1 Ã (mean over neighbours)
        out, alpha = O.gat_forward(comp, rp, ci, H, W, z, z)
        assert rel(out, (A / A.sum(1, keepdims=True)) @ H @ W) < 1e-13
    n = 11
    rp1, ci1 = O.csr_build(n, np.zeros(0, np.int32), np.zeros(0, np.int32), O.ADD_SELF_LOOPS)
    H1 = rng.uniform(-1, 1, (n, 4))
    al, ar = rng.uniform(-1, 1, 8), rng.uniform(-1, 1, 8)
    for comp in O.GAT_COMPS:       # self-loop only: alpha = I, Y = Θ
        out, alpha = O.gat_forward(comp, rp1, ci1, H1, W, al, ar)
        assert np.array_equal(alpha, np.ones(n))
        assert rel(out, H1 @ W) < 1e-14


def test_gat_reuse_equals_recompute_and_relu():
    rp, ci, _ = csr_and_dense(53, n=150, m=800)
    rng = np.random.default_rng(13)
    H, W = rng.uniform(-1, 1, (150, 12)), rng.uniform(-1, 1, (12, 20))
    al, ar = rng.uniform(-1, 1, 20), rng.uniform(-1, 1, 20)
    a = O.gat_forward(O.GAT_REUSE, rp, ci, H, W, al, ar, 1)[0]
    b = O.gat_forward(O.GAT_RECOMP, rp, ci, H, W, al, ar, 1)[0]
    assert rel(a, b) < 1e-12 and np.all(a >= 0)
    e = np.array([0.0, 1.0, -2.0])
    assert np.allclose(O.edge_softmax(np.array([0, 3]), e), np.exp(e) / np.exp(e).sum(), atol=1e-16)


# ------------------------------------------------------------------ O6 GCN backward
def loss(comp, rp, ci, H, W, G, act):
    return float((O.gcn_forward(comp, rp, ci, H, W, act)[0] * G).sum())


@pytest.mark.parametrize("comp", O.GCN_COMPS)
def test_gcn_backward_finite_differences(comp):
    rp, ci, _ = csr_and_dense(61, n=12, m=30)
    rng = np.random.default_rng(14)
    H, W = rng.uniform(-1, 1, (12, 4)), rng.uniform(-1, 1, (4, 3))
    G = rng.standard_normal((12, 3))
    for act in (0, 1):
        dH, dW = O.gcn_backward(comp, rp, ci, H, W, G, act)
        h = 1e-6
        fdW = np.zeros_like(W)
        for i in range(W.shape[0]):
            for j in range(W.shape[1]):
                Wp, Wm = W.copy(), W.copy()
                Wp[i, j] += h
                Wm[i, j] -= h
                fdW[i, j] = (loss(comp, rp, ci, H, Wp, G, act) - loss(comp, rp, ci, H, Wm, G, act)) / (2 * h)
        fdH = np.zeros_like(H)
        for i in range(H.shape[0]):
            for j in range(H.shape[1]):
                Hp, Hm = H.copy(), H.copy()
                Hp[i, j] += h
                Hm[i, j] -= h
                fdH[i, j] = (loss(comp, rp, ci, Hp, W, G, act) - loss(comp, rp, ci, Hm, W, G, act)) / (2 * h)
        assert np.max(np.abs(dW - fdW)) < 1e-7
        assert np.max(np.abs(dH - fdH)) < 1e-7


def test_gcn_backward_compositions_agree_and_identity_closed_form():
    rp, ci, _ = csr_and_dense(62, n=90, m=400, flags=O.ADD_SELF_LOOPS)  # directed: transpose matters
    rng = np.random.default_rng(15)
    H, W = rng.uniform(-1, 1, (90, 7)), rng.uniform(-1, 1, (7, 5))
    G = rng.standard_normal((90, 5))
    res = [O.gcn_backward(c, rp, ci, H, W, G, 1) for c in O.GCN_COMPS]
    for dH, dW in res[1:]:
        assert rel(dH, res[0][0]) < 1e-12 and rel(dW, res[0][1]) < 1e-12
    n = 10
    rp1, ci1 = O.csr_build(n, np.zeros(0, np.int32), np.zeros(0, np.int32), O.ADD_SELF_LOOPS)
    H1, G1 = rng.standard_normal((n, 7)), rng.standard_normal((n, 5))
    for c in O.GCN_COMPS:
        dH, dW = O.gcn_backward(c, rp1, ci1, H1, W, G1, 0)
        assert rel(dW, H1.T @ G1) < 1e-14 and rel(dH, G1 @ W.T) < 1e-14


# ------------------------------------------------------------------ GAT backward (N2, reading R22)
def gat_loss(comp, rp, ci, H, W, al, ar, G, act):
    return float((O.gat_forward(comp, rp, ci, H, W, al, ar, act)[0] * G).sum())


@pytest.mark.parametrize("comp", O.GAT_COMPS)
@pytest.mark.parametrize("flags", [O.SYMMETRIZE | O.ADD_SELF_LOOPS, O.ADD_SELF_LOOPS])
def test_gat_backward_finite_differences(comp, flags):
    """every gradient (W, H, a_l, a_r) against central differences of the pinned forward"""
    rp, ci, _ = csr_and_dense(63, n=11, m=30, flags=flags)
    rng = np.random.default_rng(16)
    H, W = rng.uniform(-1, 1, (11, 4)), rng.uniform(-1, 1, (4, 3))
    al, ar = rng.uniform(-1, 1, 3), rng.uniform(-1, 1, 3)
    G = rng.standard_normal((11, 3))
    h = 1e-6

    def fd(X, f):
        out = np.zeros_like(X)
        for idx in np.ndindex(X.shape):
            Xp, Xm = X.copy(), X.copy()
            Xp[idx] += h
            Xm[idx] -= h
            out[idx] = (f(Xp) - f(Xm)) / (2 * h)
        return out

    for act in (0, 1):
        dH, dW, dal, dar = O.gat_backward(comp, rp, ci, H, W, al, ar, G, act)
        assert np.max(np.abs(dW - fd(W, lambda x: gat_loss(comp, rp, ci, H, x, al, ar, G, act)))) < 1e-7
        assert np.max(np.abs(dH - fd(H, lambda x: gat_loss(comp, rp, ci, x, W, al, ar, G, act)))) < 1e-7
        assert np.max(np.abs(dal - fd(al, lambda x: gat_loss(comp, rp, ci, H, W, x, ar, G, act)))) < 1e-7
        assert np.max(np.abs(dar - fd(ar, lambda x: gat_loss(comp, rp, ci, H, W, al, x, G, act)))) < 1e-7


def test_gat_backward_compositions_agree_and_closed_forms():
    rp, ci, _ = csr_and_dense(64, n=80, m=500)
    rng = np.random.default_rng(17)
    H, W = rng.uniform(-1, 1, (80, 6)), rng.uniform(-1, 1, (6, 9))
    al, ar = rng.uniform(-1, 1, 9), rng.uniform(-1, 1, 9)
    G = rng.standard_normal((80, 9))
    a = O.gat_backward(O.GAT_REUSE, rp, ci, H, W, al, ar, G, 1)
    b = O.gat_backward(O.GAT_RECOMP, rp, ci, H, W, al, ar, G, 1)
    for x, y in zip(a, b):
        assert rel(x, y) < 1e-12
    # need_dH=False leaves the parameter gradients unchanged
    c = O.gat_backward(O.GAT_REUSE, rp, ci, H, W, al, ar, G, 1, need_dH=False)
    assert c[0] is None and rel(c[1], a[1]) < 1e-15 and rel(c[2], a[2]) < 1e-15
    # self-loop-only graph: α = I, so Y = Θ, dW = Hᵀ G, dH = G Wᵀ and the scores get no gradient
    n = 10
    rp1, ci1 = O.csr_build(n, np.zeros(0, np.int32), np.zeros(0, np.int32), O.ADD_SELF_LOOPS)
    H1, G1 = rng.standard_normal((n, 6)), rng.standard_normal((n, 9))
    for comp in O.GAT_COMPS:
        dH, dW, dal, dar = O.gat_backward(comp, rp1, ci1, H1, W, al, ar, G1, 0)
        assert rel(dW, H1.T @ G1) < 1e-14 and rel(dH, G1 @ W.T) < 1e-14
        assert np.all(dal == 0) and np.all(dar == 0)
    # a_l = a_r = 0: uniform attention α = D⁻¹Ã; dW and dH are the mean-aggregation GCN's
    z = np.zeros(9)
    dH, dW, dal, dar = O.gat_backward(O.GAT_REUSE, rp, ci, H, W, z, z, G, 0)
    A = np.zeros((80, 80))
    for r in range(80):
        A[r, ci[rp[r]:rp[r + 1]]] = 1.0 / (rp[r + 1] - rp[r])
    assert rel(dW, (A @ H).T @ G) < 1e-12 and rel(dH, A.T @ G @ W.T) < 1e-12


@pytest.mark.parametrize("K1,K2", [(5, 7), (7, 5)])
def test_gat_backward_magnitude_bounds_and_closed_form(K1, K2):
    """the tolerance scale dominates every gradient entry (triangle inequality) and equals the
    gradient when nothing can cancel (H, W, G >= 0, a_l = a_r = 0: dW = (αH)ᵀG, dH = αᵀ G Wᵀ)"""
    rp, ci, _ = csr_and_dense(65, n=60, m=300)
    rng = np.random.default_rng(18)
    H, W = rng.uniform(-1, 1, (60, K1)), rng.uniform(-1, 1, (K1, K2))
    al, ar = rng.uniform(-1, 1, K2), rng.uniform(-1, 1, K2)
    G = rng.standard_normal((60, K2))
    for comp in O.GAT_COMPS:
        for act in (0, 1):
            g = O.gat_backward(comp, rp, ci, H, W, al, ar, G, act)
            m = O.gat_backward_magnitude(comp, rp, ci, H, W, al, ar, G, act)
            for x, y in zip(g, m):
                assert np.all(np.abs(x) <= y * (1 + 1e-12) + 1e-300)
    Hp, Wp, Gp, z = np.abs(H), np.abs(W), np.abs(G), np.zeros(K2)
    for comp in O.GAT_COMPS:
        g = O.gat_backward(comp, rp, ci, Hp, Wp, z, z, Gp, 0)
        m = O.gat_backward_magnitude(comp, rp, ci, Hp, Wp, z, z, Gp, 0)
        assert rel(m[0], g[0]) < 1e-13 and rel(m[1], g[1]) < 1e-13


# ------------------------------------------------------------------ N3: SGC / TAGCN / GIN (reading R23)
def dense_S(A):
    deg = A.sum(1)
    dm = np.where(deg > 0, 1.0 / np.sqrt(np.where(deg > 0, deg, 1)), 0.0)
    return np.diag(dm) @ A @ np.diag(dm)


@pytest.mark.parametrize("comp", O.SGC_COMPS)
@pytest.mark.parametrize("hops", [0, 1, 3])
def test_sgc_equals_dense_power(comp, hops):
    rp, ci, A = csr_and_dense(71)
    rng = np.random.default_rng(21)
    H, W = rng.uniform(-1, 1, (29, 6)), rng.uniform(-1, 1, (6, 4))
    S = dense_S(A)
    for act in (0, 1):
        Y = np.linalg.matrix_power(S, hops) @ H @ W
        assert rel(O.sgc_forward(comp, rp, ci, H, W, hops, act), np.maximum(Y, 0) if act else Y) < 1e-12


def test_sgc_one_hop_is_gcn():
    rp, ci, _ = csr_and_dense(72)
    rng = np.random.default_rng(22)
    H, W = rng.uniform(-1, 1, (29, 5)), rng.uniform(-1, 1, (5, 7))
    for c_sgc, c_gcn in zip(O.SGC_COMPS, O.GCN_COMPS):
        assert rel(O.sgc_forward(c_sgc, rp, ci, H, W, 1, 1), O.gcn_forward(c_gcn, rp, ci, H, W, 1)[0]) < 1e-12


@pytest.mark.parametrize("comp", O.TAGCN_COMPS)
@pytest.mark.parametrize("hops", [0, 1, 2, 3])
def test_tagcn_equals_dense_polynomial(comp, hops):
    rp, ci, A = csr_and_dense(73)
    rng = np.random.default_rng(23)
    H = rng.uniform(-1, 1, (29, 5))
    Ws = rng.uniform(-1, 1, (hops + 1, 5, 3))
    S = dense_S(A)
    Y = sum(np.linalg.matrix_power(S, j) @ H @ Ws[j] for j in range(hops + 1))
    for act in (0, 1):
        assert rel(O.tagcn_forward(comp, rp, ci, H, Ws, act), np.maximum(Y, 0) if act else Y) < 1e-12
    # only W_0 nonzero: a plain matmul, whatever the graph
    W0 = np.zeros_like(Ws)
    W0[0] = Ws[0]
    assert rel(O.tagcn_forward(comp, rp, ci, H, W0, 0), H @ Ws[0]) < 1e-14


@pytest.mark.parametrize("comp", O.GIN_COMPS)
def test_gin_equals_dense_mlp(comp):
    n = 31
    s, d = synth.random_small(n, 120, 74)
    rp, ci = O.csr_build(n, s, d, O.SYMMETRIZE | O.ADD_SELF_LOOPS)
    A0 = dense_adj(n, s.numpy(), d.numpy(), True, False)
    np.fill_diagonal(A0, 0.0)                  # neighbours j != i: GIN's own term is (1 + eps) H_i
    rng = np.random.default_rng(24)
    H, W1, W2 = rng.uniform(-1, 1, (n, 6)), rng.uniform(-1, 1, (6, 9)), rng.uniform(-1, 1, (9, 4))
    for eps in (0.0, 0.37, -0.5):
        agg = (1 + eps) * H + A0 @ H
        Y = np.maximum(agg @ W1, 0) @ W2
        for act in (0, 1):
            got = O.gin_forward(comp, rp, ci, H, W1, W2, eps, act)
            assert rel(got, np.maximum(Y, 0) if act else Y) < 1e-12
    # self-loop-only graph: agg = (1 + eps) H
    rp1, ci1 = O.csr_build(n, np.zeros(0, np.int32), np.zeros(0, np.int32), O.ADD_SELF_LOOPS)
    assert rel(O.gin_forward(comp, rp1, ci1, H, W1, W2, 0.25, 0), np.maximum(1.25 * H @ W1, 0) @ W2) < 1e-14


# ------------------------------------------------------------------ generators
def test_generator_is_device_independent_and_exact():
    a = synth.uniform_pm1(3, 4, (1000,))
    assert a.dtype.name == "float32" if hasattr(a.dtype, "name") else True
    v = a.numpy()
    assert np.all((v >= -1) & (v < 1))
    assert np.array_equal(v, (np.round((v + 1) * 2 ** 23) / 2 ** 23 - 1).astype(np.float32))
    # splitmix64 against a pure-Python reference
    def ref(x):
        m = (1 << 64) - 1
        z = (x + 0x9E3779B97F4A7C15) & m
        z = ((z ^ (z >> 30)) * 0xBF58476D1CE4E5B9) & m
        z = ((z ^ (z >> 27)) * 0x94D049BB133111EB) & m
        return z ^ (z >> 31)
    import torch
    xs = torch.tensor([0, 1, 2, 12345678901234, -5], dtype=torch.int64)
    got = [int(v) & ((1 << 64) - 1) for v in synth.splitmix64(xs)]
    assert got == [ref(int(x) & ((1 << 64) - 1)) for x in xs]


def test_workload_shapes_match_paper_table2():
    g = json.load(open(os.path.join(GOLDEN, "paper_shapes.json")))
    for name, row in g["graphs"].items():
        w = synth.WORKLOADS[name]
        assert w.n == row["nodes"], name
