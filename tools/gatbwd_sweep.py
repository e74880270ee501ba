"""GAT backward micro-sweep: time gat_bwd_a / gat_bwd_b of one layer per GRANII_GATBWD="LPG,NJ,U" setting.
usage: python tools/gatbwd_sweep.py [graph] ; env CASES="comp:K1:K2[:dH];..." TUNES="def;16,2,2;...";
dH = 0 runs the backward without the input gradient (a RECOMP input layer: pass A + the der-only passes)."""
import os
import sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_cgo_lenadorasgytm26_b200 import granii as G, synth
from paper_conf_cgo_lenadorasgytm26_b200.model import GNN, LayerSpec, alloc2d

dev = torch.device("cuda:0")
wname = sys.argv[1] if len(sys.argv) > 1 else "products"
w = synth.WORKLOADS[wname]
s, d = w.edges(0, device=dev)
g = G.granii_graph_csr_create(w.n, s, d, G.ADD_SELF_LOOPS | (G.SYMMETRIZE if w.symmetrize else 0))
print("graph", wname, "nnz", g.nnz, flush=True)
for case in os.environ.get("CASES", "17:100:256;16:256:47").split(";"):
    f = [int(x) for x in case.split(":")]
    comp, K1, K2 = f[:3]
    need = bool(f[3]) if len(f) > 3 else True
    H = alloc2d(w.n, K1, dev)
    H.copy_(synth.features(1, w.n, K1).to(dev))
    W = synth.glorot(2, 3, K1, K2, (K1, K2)).to(dev)
    al = synth.uniform_pm1(4, 1, (K2,)).to(dev)
    ar = synth.uniform_pm1(4, 2, (K2,)).to(dev)
    net = GNN(g, [LayerSpec(G.GAT, K1, K2, G.ACT_RELU, comp=comp, W=W, a_l=al, a_r=ar)], dev)
    net.forward(H)
    dout = alloc2d(w.n, K2, dev)
    dout.copy_(synth.uniform_pm1(3, 7, (w.n, K2)).to(dev))
    for tune in os.environ.get("TUNES", "def;16,2,2;16,2,4;32,1,2;32,1,4;8,2,4;16,1,4").split(";"):
        os.environ.pop("GRANII_GATBWD", None)
        if tune != "def":
            os.environ["GRANII_GATBWD"] = tune
        net.backward(dout, need_input_grad=need)
        torch.cuda.synchronize()
        G.granii_profile_enable(True)
        for _ in range(3):
            net.backward(dout, need_input_grad=need)
        torch.cuda.synchronize()
        p = G.granii_profile_read()
        G.granii_profile_enable(False)
        row = {k: round(v["ms"] / 3, 3) for k, v in p.items()}
        print(f"{G.COMP_NAMES[comp]} {K1}->{K2} dH={int(need)} tune={tune:12s} " +
              " ".join(f"{k}={v}" for k, v in sorted(row.items())), flush=True)
