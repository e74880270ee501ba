#!/usr/bin/env python
"""Per-primitive view of one selection: for a workload graph and one layer shape, time every
candidate composition (forward, + backward with --train) through the library's tracer and print
measured ms per primitive next to the selector's predicted totals.

    python tools/explain_select.py pubmed gat 64 256 [--train] [--input-layer]
"""
import argparse
import os
import sys

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_cgo_lenadorasgytm26_b200 import granii as G, synth  # noqa: E402
from paper_conf_cgo_lenadorasgytm26_b200.model import DEFAULT_CALIB, GNN, LayerSpec, alloc2d  # noqa: E402

DEV = torch.device("cuda:0")


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("graph")
    ap.add_argument("model", choices=["gcn", "gat"])
    ap.add_argument("K1", type=int)
    ap.add_argument("K2", type=int)
    ap.add_argument("--train", action="store_true")
    ap.add_argument("--input-layer", action="store_true")
    a = ap.parse_args()
    w = synth.WORKLOADS[a.graph]
    s, d = w.edges(0, DEV)
    g = G.granii_graph_csr_create(w.n, s, d, G.ADD_SELF_LOOPS | (G.SYMMETRIZE if w.symmetrize else 0))
    model = G.GCN if a.model == "gcn" else G.GAT
    fl = (G.SELECT_TRAINING | (G.SELECT_INPUT_LAYER if a.input_layer else 0)) if a.train else 0
    sel, pred = G.granii_select(g, model, a.K1, a.K2, DEFAULT_CALIB, fl | G.SELECT_NO_PREFILTER)
    H = alloc2d(g.n_rows, a.K1, DEV, fill=0.5)
    gup = alloc2d(g.n_rows, a.K2, DEV, fill=0.01)
    W = synth.glorot(2, 0, a.K1, a.K2, (a.K1, a.K2), device=DEV).contiguous()
    al = synth.uniform_pm1(3, 0, (a.K2,), device=DEV)
    ar = synth.uniform_pm1(3, 1, (a.K2,), device=DEV)
    print(f"{a.graph} rows={g.n_rows} nnz={g.nnz} {a.model} {a.K1}->{a.K2} train={a.train} "
          f"selected={G.COMP_NAMES[sel]}")
    for c in G.COMPS[model]:
        net = GNN(g, [LayerSpec(model, a.K1, a.K2, G.ACT_RELU, comp=c, W=W, a_l=al, a_r=ar)], DEV)

        def fn():
            net.forward(H)
            if a.train:
                net.backward(gup, need_input_grad=not a.input_layer)
        for _ in range(3):
            fn()
        torch.cuda.synchronize()
        G.granii_profile_enable(True)
        reps = 10
        for _ in range(reps):
            fn()
        torch.cuda.synchronize()
        prof = G.granii_profile_read()
        G.granii_profile_enable(False)
        tot = sum(v["ms"] for v in prof.values()) / reps
        parts = ", ".join(f"{k} {v['ms'] / reps:.3f} ({v['calls'] // reps})" for k, v in sorted(prof.items()))
        print(f"  {G.COMP_NAMES[c]:12s} measured {tot:.3f} ms  predicted {pred.get(c, float('nan')):.3f}  | {parts}")


if __name__ == "__main__":
    main()
