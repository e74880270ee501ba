"""Small end-to-end workload for compute-sanitizer (memcheck / racecheck / initcheck / synccheck):
every GCN and GAT composition forward + backward on a sparse (group-per-row) and a dense
(warp-per-row, hub segments) graph, the fused and unfused attention (both K = 1 SDDMM kernels), directed
backward over the
kept transpose, the primitives, both tcgen05 GEMMs, SGC / TAGCN / GIN, softmax-xent + SGD.
Shapes are tiny so the instrumented run stays in minutes.  Exit code 0 = all calls returned OK."""
import os
import sys

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_cgo_lenadorasgytm26_b200 import granii as G  # noqa: E402
from paper_conf_cgo_lenadorasgytm26_b200 import synth  # noqa: E402
from paper_conf_cgo_lenadorasgytm26_b200.model import GNN, LayerSpec, alloc2d  # noqa: E402

dev = torch.device("cuda:0")
os.environ.setdefault("GRANII_SEG", "64")       # hub segments on the dense graph


def graph(kind):
    if kind == "sparse":
        n = 600
        s, d = synth.chung_lu(n, 1500, 2.5, seed=2)
        fl = G.ADD_SELF_LOOPS | G.SYMMETRIZE
    elif kind == "dense":
        n = 400
        s, d = synth.chung_lu(n, 12000, 2.1, seed=3, max_w_frac=0.05)
        fl = G.ADD_SELF_LOOPS | G.SYMMETRIZE
    else:
        n = 500
        s, d = synth.rmat(n, 4000, 0.57, 0.19, 0.19, seed=4)
        fl = G.ADD_SELF_LOOPS | G.BUILD_TRANSPOSE
    return n, G.granii_graph_csr_create(n, s.to(dev), d.to(dev), fl)


def main():
    torch.cuda.set_device(dev)
    for kind in ("sparse", "dense", "directed"):
        n, g = graph(kind)
        K1, K2 = 40, 24
        H = alloc2d(n, K1, dev)
        H.copy_(synth.features(1, n, K1).to(dev))
        W = synth.glorot(2, 3, K1, K2, (K1, K2)).to(dev)
        up = alloc2d(n, K2, dev)
        up.copy_(synth.uniform_pm1(3, 7, (n, K2)).to(dev))
        al = synth.uniform_pm1(4, 1, (K2,)).to(dev)
        ar = synth.uniform_pm1(4, 2, (K2,)).to(dev)
        for comp in G.GCN_COMPS:
            net = GNN(g, [LayerSpec(G.GCN, K1, K2, G.ACT_RELU, comp=comp, W=W.clone())], dev)
            net.forward(H)
            net.backward(up, need_input_grad=True)
        for fused, tile in (("1", "0"), ("0", "0"), ("0", "1")):   # tile: the entry-tile K = 1 SDDMM
            os.environ["GRANII_GAT_FUSED"] = fused
            os.environ["GRANII_SDDMM_TILE"] = tile
            for comp in G.GAT_COMPS:
                net = GNN(g, [LayerSpec(G.GAT, K1, K2, G.ACT_RELU, comp=comp, W=W.clone(), a_l=al, a_r=ar)], dev)
                net.forward(H)
                net.backward(up, need_input_grad=True)
        if kind != "directed":
            for comp in (32, 35):
                GNN(g, [LayerSpec(G.SGC, K1, K2, 0, comp=comp, W=W, hops=2)], dev).forward(H)
            Ws = synth.glorot(5, 2, K1, K2, (3, K1, K2)).to(dev).contiguous()
            for comp in (48, 51):
                GNN(g, [LayerSpec(G.TAGCN, K1, K2, 0, comp=comp, W=Ws, hops=2)], dev).forward(H)
            W1 = synth.glorot(6, 2, K1, 32, (K1, 32)).to(dev)
            W2 = synth.glorot(6, 3, 32, K2, (32, K2)).to(dev)
            for comp in (64, 67):
                GNN(g, [LayerSpec(G.GIN, K1, K2, 1, comp=comp, W=W1, eps=0.1, Kh=32, W2=W2)], dev).forward(H)
        # two-layer training step with the selector (refine off: no timing inside the sanitizer)
        spec = [LayerSpec(G.GCN, K1, 32, G.ACT_RELU, W=synth.glorot(7, 1, K1, 32, (K1, 32)).to(dev)),
                LayerSpec(G.GCN, 32, 7, G.ACT_NONE, W=synth.glorot(7, 2, 32, 7, (32, 7)).to(dev))]
        net = GNN(g, spec, dev, select_flags=0, training=True)
        y = synth.labels(8, n, 7).to(dev)
        dl = alloc2d(n, 7, dev)
        loss = torch.zeros(n, device=dev)
        net.train_step(H, y, n, 0.01, dl, loss)
        torch.cuda.synchronize()
        print(f"{kind}: ok", flush=True)
    print("sanitize_run: all calls OK")


if __name__ == "__main__":
    main()
