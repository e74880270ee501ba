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


def build(G, name):
    w = synth.WORKLOADS[name]
    src, dst = w.edges(seed=0, device=DEV)
    flags = G.ADD_SELF_LOOPS | (G.SYMMETRIZE if w.symmetrize else 0)
    g = G.granii_graph_csr_create(w.n, src, dst, flags)
    rp, ci = O.csr_build(w.n, src.cpu(), dst.cpu(), flags)
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
    MH1 = O.spmm(rp, ci, O.sddmm(rp, ci, O.dinv(rp), O.dinv(rp)), H1)
    dW2 = O.gemm(MH1, gup.cpu().numpy(), ta=True)     # identity activation on the last layer
    d = np.abs(net.dW[1].cpu().numpy() - dW2)
    assert float((d.max(1) / np.abs(dW2).max(1)).max()) <= TOL


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
