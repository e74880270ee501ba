"""Where does the full-size products GAT backward's normwise dW / da error come from?  Runs the
test_products_gat_training_fullsize setting for one layer (argv[1] = 0 or 1), the fp64 oracle over all
rows, and reports: per-row relative error of dΘ (REUSE: recovered from dH = dΘ Wᵀ by least squares;
layer 0 RECOMP: del from da is not recoverable, so only the da / dW totals), its dependence on the row
degree, and which rows carry the dW error Hᵀ(dΘ_gpu - dΘ_ref)."""
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))
import oracle as O  # noqa: E402
import bench  # noqa: E402
from paper_conf_cgo_lenadorasgytm26_b200 import granii as G, synth  # noqa: E402
from paper_conf_cgo_lenadorasgytm26_b200.model import GNN, LayerSpec, alloc2d  # noqa: E402

DEV = torch.device("cuda:0")
layer = int(sys.argv[1]) if len(sys.argv) > 1 else 1
w = synth.WORKLOADS["products"]
src, dst = w.edges(seed=0, device=DEV)
g = G.granii_graph_csr_create(w.n, src, dst, G.ADD_SELF_LOOPS | G.SYMMETRIZE)
rp, ci = G.granii_graph_export_csr(g)
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
    U[torch.from_numpy(np.abs(Y) < 1e-4 * np.abs(Y).max())] = 0.0
    del Y
if os.environ.get("R27", "1") == "1":
    from test_gpu_parity import leaky_ambiguous_rows
    amb = leaky_ambiguous_rows(rp, ci, Hn, Wn, al, ar)
    print(f"R27: {amb.shape[0]} rows with an ambiguous LeakyReLU' decision zeroed", flush=True)
    U[torch.from_numpy(amb)] = 0.0
net = GNN(g, [LayerSpec(G.GAT, K1, K2, act, G.ATTN_ADDITIVE, comp=L.comp, W=L.W, a_l=L.a_l, a_r=L.a_r)], DEV)
net.forward(H)
Ud = alloc2d(w.n, K2, DEV)
Ud.copy_(U)
dH = net.backward(Ud, need_input_grad=need_dH)
torch.cuda.synchronize()
ref = O.gat_backward(L.comp, rp, ci, Hn, Wn, al, ar, U, act, need_dH=need_dH)
got = (dH, net.dW[0], net.da[0][0], net.da[0][1])
for nm, y, r in zip(("dH", "dW", "da_l", "da_r"), got, ref):
    if y is None or r is None:
        continue
    y = np.atleast_2d(y.cpu().numpy().astype(np.float64))
    r = np.atleast_2d(r)
    print(f"{G.COMP_NAMES[L.comp]} {nm}: normwise {np.abs(y - r).max() / np.abs(r).max():.3e}", flush=True)
deg = np.diff(rp)
if need_dH:
    Wd = Wn.astype(np.float64)
    P = np.linalg.pinv(Wd.T)  # dΘ = dH (Wᵀ)^+
    dth = dH.cpu().numpy().astype(np.float64) @ P
    dthr = ref[0] @ P
    e = np.abs(dth - dthr).max(1) / np.maximum(np.abs(dthr).max(1), 1e-30)
    for lo, hi in ((1, 8), (8, 32), (32, 128), (128, 512), (512, 2048), (2048, 10 ** 9)):
        m = (deg >= lo) & (deg < hi)
        if m.any():
            print(f"deg [{lo},{hi}): rows {m.sum()}  dTheta row rel err median {np.median(e[m]):.2e} "
                  f"p99 {np.quantile(e[m], 0.99):.2e} max {e[m].max():.2e}", flush=True)
    D = dth - dthr
    dWe = Hn.astype(np.float64).T @ D
    print(f"dW error recomputed from dTheta: normwise {np.abs(dWe).max() / np.abs(ref[1]).max():.3e}")
    # contribution of the hub rows (top 1 % by degree) vs the rest
    top = deg >= np.quantile(deg, 0.99)
    for nm, m in (("top1%", top), ("rest", ~top)):
        c = Hn[m].astype(np.float64).T @ D[m]
        print(f"  {nm}: {np.abs(c).max() / np.abs(ref[1]).max():.3e}")
    # mean (systematic) vs fluctuating part of the dΘ error
    rel = D / np.maximum(np.abs(dthr), 1e-30)
    print(f"dTheta signed rel err mean {np.mean(np.sign(dthr) * D / np.maximum(np.abs(dthr).max(1, keepdims=True), 1e-30)):.3e}")
