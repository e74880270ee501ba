"""Parity at BASELINE.json's full sizes, in bench.py's launch configuration (-m gpu).

The graphs, features and weights are the bench's (same seeds, same generators),
the GPU runs the same multi-layer model with the compositions granii_select
picks, and the fp64 oracle is evaluated one row at a time on a sample: 4096
random rows plus the 64 highest-degree rows (hub rows exercise the segmented
path).  The CSR is compared bit-exactly in full.  Tolerance: R19 (row-normwise
relative error <= 1e-4).
"""
import numpy as np
import pytest
import torch

import oracle as O
from paper_conf_cgo_lenadorasgytm26_b200 import synth

pytestmark = pytest.mark.gpu
DEV = torch.device("cuda:0") if torch.cuda.is_available() else None
TOL = 1e-4


def rowerr(y, r):
    d = np.abs(np.asarray(y, np.float64) - r).max(1)
    a = np.abs(r).max(1)
    return float((d / np.maximum(a, 1e-6 * np.abs(r).max())).max())


def sample_rows(rp, n_rand=4096, n_top=64, seed=0):
    deg = np.diff(rp)
    rng = np.random.default_rng(seed)
    top = np.argsort(-deg, kind="stable")[:n_top]
    return np.unique(np.concatenate([rng.choice(rp.shape[0] - 1, n_rand, replace=False), top]))


@pytest.fixture(scope="module")
def G():
    from paper_conf_cgo_lenadorasgytm26_b200 import granii
    return granii


_graphs = {}


def build(G, name):
    if name in _graphs:
        return _graphs[name]
    w = synth.WORKLOADS[name]
    src, dst = w.edges(seed=0, device=DEV)
    flags = G.ADD_SELF_LOOPS | (G.SYMMETRIZE if w.symmetrize else 0)
    g = G.granii_graph_csr_create(w.n, src, dst, flags)
    rp, ci = O.csr_build(w.n, src.cpu(), dst.cpu(), flags)
    _graphs.clear()                      # one full-size graph resident at a time
    _graphs[name] = (w, g, rp, ci)
    return w, g, rp, ci


def test_reddit_training_step_fullsize(G):
    """C4: Reddit-shaped graph (~118M stored entries), GCN 602 -> 256 -> 41 as in bench.py."""
    import bench
    from paper_conf_cgo_lenadorasgytm26_b200.model import alloc2d
    w, g, rp, ci = build(G, "reddit")
    grp, gci = G.granii_graph_export_csr(g)
    assert np.array_equal(grp, rp) and np.array_equal(gci, ci), "full-size CSR must be bit-exact"
    spec = bench.WORKLOADS["reddit-gcn2-train"]
    net = bench.build_model(G, None, spec, g, DEV, None)
    H = alloc2d(w.n, 602, DEV)
    H.copy_(synth.features(1, w.n, 602, device=DEV))
    W1 = net.layers[0].W.cpu().numpy().astype(np.float64)
    W2 = net.layers[1].W.cpu().numpy().astype(np.float64)
    out = net.forward(H)
    torch.cuda.synchronize()
    rows = sample_rows(rp)
    deg = np.diff(rp)
    Hn = H.cpu().numpy()
    # layer 1 at every row (the second layer's sampled rows need all their neighbours)
    H1 = O.gcn_rows(np.arange(w.n), rp, ci, deg, Hn, W1, 1)
    assert rowerr(net.outs[0].cpu().numpy()[rows], H1[rows]) <= TOL
    ref2 = O.gcn_rows(rows, rp, ci, deg, H1, W2, 0)
    assert rowerr(out.cpu().numpy()[rows], ref2) <= TOL
    # backward of the last layer: dW2 = (M H1)ᵀ dY over ALL rows (a full reduction)
    gup = synth.uniform_pm1(5, 1, (w.n, 41), device=DEV)
    gpad = alloc2d(w.n, 41, DEV)
    gpad.copy_(gup)
    net.backward(gpad)
    torch.cuda.synchronize()
    nval = O.sddmm(rp, ci, O.dinv(rp), O.dinv(rp))
    MH1 = O.spmm(rp, ci, nval, H1)
    dW2 = O.gemm(MH1, gup.cpu().numpy(), ta=True)     # identity activation on the last layer
    d = np.abs(net.dW[1].cpu().numpy() - dW2)
    assert float((d.max(1) / np.abs(dW2).max(1)).max()) <= TOL
    # the gradient handed to layer 1: dL/dH1 = Mᵀ dY2 W2ᵀ (M symmetric), every row
    dH1 = O.gemm(O.spmm(rp, ci, nval, gup.cpu().numpy()), W2, tb=True)
    assert rowerr(net.grads_out[0].cpu().numpy(), dH1) <= TOL


def test_reddit_layer1_backward_fullsize(G):
    """C4 layer 1 as the timed step runs it: GCN 602 -> 256 + ReLU under the composition the
    selector picks for training (input layer: no dH), i.e. the K=256 transpose aggregation with its
    L2-resident column slices and hub segments, then dW1 = (M H)ᵀ dY1 (602 x 256) reduced over all
    232,965 rows, against oracle_gcn_backward.  The upstream gradient is random and zeroed where
    |Y1| is within rounding of 0, so the ReLU' decision is unique (R20)."""
    import bench
    from paper_conf_cgo_lenadorasgytm26_b200.model import GNN, LayerSpec, alloc2d
    w, g, rp, ci = build(G, "reddit")
    spec = bench.WORKLOADS["reddit-gcn2-train"]
    full = bench.build_model(G, None, spec, g, DEV, None)
    L0 = full.layers[0]
    del full
    H = alloc2d(w.n, 602, DEV)
    H.copy_(synth.features(1, w.n, 602, device=DEV))
    Hn = H.cpu().numpy()
    W1 = L0.W.cpu().numpy().astype(np.float64)
    Y1 = O.gcn_rows(np.arange(w.n), rp, ci, np.diff(rp), Hn, W1, 0)       # pre-activation, fp64
    U = synth.uniform_pm1(6, 1, (w.n, 256))
    U[torch.from_numpy(np.abs(Y1) < 1e-4 * np.abs(Y1).max())] = 0.0
    net = GNN(g, [LayerSpec(G.GCN, 602, 256, G.ACT_RELU, comp=L0.comp, W=L0.W)], DEV)
    net.forward(H)
    Ud = alloc2d(w.n, 256, DEV)
    Ud.copy_(U)
    assert net.backward(Ud) is None                  # input layer: no dH, as in the step
    torch.cuda.synchronize()
    _, dW1 = O.gcn_backward(L0.comp, rp, ci, Hn, W1, U, 1, need_dH=False)
    assert rowerr(net.dW[0].cpu().numpy(), dW1) <= TOL, G.COMP_NAMES[L0.comp]


@pytest.mark.parametrize("model", ["gcn", "gat"])
def test_products_inference_fullsize(G, model):
    """C5: ogbn-products-shaped graph (~126M stored entries, 2.45M nodes), layer 1 (100 -> 256)."""
    import bench
    from paper_conf_cgo_lenadorasgytm26_b200.model import alloc2d
    w, g, rp, ci = build(G, "products")
    spec = dict(bench.WORKLOADS[f"products-{model}2-infer"])
    spec["dims"] = [100, 256]
    net = bench.build_model(G, None, spec, g, DEV, None)
    net.layers[0].act = G.ACT_RELU
    H = alloc2d(w.n, 100, DEV)
    H.copy_(synth.features(1, w.n, 100, device=DEV))
    out = net.forward(H)
    torch.cuda.synchronize()
    rows = sample_rows(rp)
    L = net.layers[0]
    Hn, Wn = H.cpu().numpy(), L.W.cpu().numpy()
    if model == "gcn":
        ref = O.gcn_rows(rows, rp, ci, np.diff(rp), Hn, Wn, 1)
    else:
        ref = O.gat_rows(rows, rp, ci, Hn, Wn, L.a_l.cpu().numpy(), L.a_r.cpu().numpy(), 1)
    assert rowerr(out.cpu().numpy()[rows], ref) <= TOL, G.COMP_NAMES[L.comp]


@pytest.mark.parametrize("layer", [0, 1])
def test_products_gat_training_fullsize(G, layer):
    """C5 GAT training (products-gat2-train, 100 -> 256 -> 47): each layer's backward at full size
    under the composition the bench selects, one layer at a time so the ReLU' decision can be made
    unique (R20; R27 for LeakyReLU' on the scores): dW, da_l, da_r (reductions over all 2.45M rows)
    and, for the second layer (which the step differentiates with respect to its input), dH on 4,096
    random + 64 hub rows, against
    oracle_gat_backward with the R22 tolerance (gat_grad_ok).  These are the pass A / pass B
    shapes (K = 100 for RECOMP's dT H rows, K = 47 for REUSE's dY Θ rows) chosen only at this scale."""
    import bench
    from test_gpu_parity import gat_grad_ok, leaky_ambiguous_rows
    from paper_conf_cgo_lenadorasgytm26_b200.model import GNN, LayerSpec, alloc2d
    w, g, rp, ci = build(G, "products")
    spec = bench.WORKLOADS["products-gat2-train"]
    full = bench.build_model(G, None, spec, g, DEV, None)
    L = full.layers[layer]
    del full
    K1, K2 = L.K1, L.K2
    act = G.ACT_RELU if layer == 0 else G.ACT_NONE
    need_dH = layer > 0
    H = alloc2d(w.n, K1, DEV)
    H.copy_(synth.features(10 + layer, w.n, K1, device=DEV))
    Hn = H.cpu().numpy()
    Wn, al, ar = (x.cpu().numpy() for x in (L.W, L.a_l, L.a_r))
    U = synth.uniform_pm1(7, layer, (w.n, K2))
    if act:
        Y, _ = O.gat_forward(L.comp, rp, ci, Hn, Wn, al, ar, 0)
        U[torch.from_numpy(np.abs(Y) < 1e-4 * np.abs(Y).max())] = 0.0      # R20
        del Y
    amb = leaky_ambiguous_rows(rp, ci, Hn, Wn, al, ar)                       # R27
    assert amb.shape[0] < 0.005 * w.n   # 3,639 / 3,825 rows of 2.45 M (layers 0 / 1)
    U[torch.from_numpy(amb)] = 0.0
    net = GNN(g, [LayerSpec(G.GAT, K1, K2, act, G.ATTN_ADDITIVE, comp=L.comp, W=L.W, a_l=L.a_l, a_r=L.a_r)], DEV)
    net.forward(H)
    Ud = alloc2d(w.n, K2, DEV)
    Ud.copy_(U)
    dH = net.backward(Ud, need_input_grad=need_dH)
    torch.cuda.synchronize()
    rows = sample_rows(rp)
    ref = O.gat_backward(L.comp, rp, ci, Hn, Wn, al, ar, U, act, need_dH=need_dH)
    mag = O.gat_backward_magnitude(L.comp, rp, ci, Hn, Wn, al, ar, U, act, need_dH=need_dH)
    got = (dH, net.dW[0], net.da[0][0], net.da[0][1])
    for nm, y, r, m in zip(("dH", "dW", "da_l", "da_r"), got, ref, mag):
        if nm == "dH":
            if not need_dH:
                continue
            y, r, m = y.cpu().numpy()[rows], r[rows], m[rows]
        else:
            y = y.cpu().numpy()
        assert gat_grad_ok(y, r, m), (G.COMP_NAMES[L.comp], nm)


def test_products_sddmm_entry_tiles_fullsize(G):
    """C5 K = 1 SDDMM at full size: the products-shaped graph (130 M stored entries) is where the
    entry-tile kernel is chosen (average degree < 128, >= 16 Mi entries).  Normalisation
    scores Ñ = D̃^-½ Ã D̃^-½ (Eq. 3) and the GAT scores + row softmax (Eq. 4, reading R8) on 4,096 random
    + 64 hub rows -- the hubs span many 4096-entry tiles, so their softmax goes through the cut-row
    combine -- against oracle_sddmm / oracle_edge_softmax over the sampled rows' CSR."""
    w, g, rp, ci = build(G, "products")
    rows = sample_rows(rp, seed=3)
    deg = np.diff(rp)
    assert deg[rows].max() > 3 * 4096       # a hub of the sample crosses several tiles
    srp = np.concatenate([[0], np.cumsum(deg[rows])]).astype(np.int64)
    sel = np.concatenate([np.arange(rp[r], rp[r + 1]) for r in rows])
    sci = ci[sel]
    dinv = O.dinv(rp)
    dv = torch.tensor(dinv, dtype=torch.float32, device=DEV)
    out = torch.empty(g.nnz, device=DEV)
    G.granii_sddmm(g, G.SDDMM_DOT, dv, 1, dv, 1, 1, 1.0, out)
    torch.cuda.synchronize()
    got = out.cpu().numpy()[sel]
    ref = O.sddmm(srp, sci, dinv[rows], dinv)
    assert float(np.max(np.abs(got - ref) / np.abs(ref))) <= TOL
    el = synth.uniform_pm1(35, 1, (w.n,)) * 4
    er = synth.uniform_pm1(35, 2, (w.n,)) * 4
    G.granii_sddmm(g, G.SDDMM_ADD | G.SDDMM_LEAKYRELU | G.SDDMM_ROW_SOFTMAX, el.to(DEV), 1, er.to(DEV), 1, 1, 1.0,
                   out)
    torch.cuda.synchronize()
    got = out.cpu().numpy()[sel].astype(np.float64)
    e = np.repeat(el.numpy().astype(np.float64)[rows], deg[rows]) + er.numpy().astype(np.float64)[sci]
    ref = O.edge_softmax(srp, np.where(e > 0, e, 0.2 * e))
    d = np.maximum.reduceat(np.abs(got - ref), srp[:-1])
    a = np.maximum.reduceat(np.abs(ref), srp[:-1])
    assert float(np.max(d / a)) <= TOL
    sums = np.add.reduceat(got, srp[:-1])
    assert np.abs(sums - 1).max() < 1e-5
