"""Normalisation SDDMM (K = 1 DOT of D^-1/2, D^-1/2) timing on the workload graphs: one line per graph."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_cgo_lenadorasgytm26_b200 import granii as G, synth
dev = torch.device("cuda:0")
for name in ("pubmed", "arxiv", "reddit", "products"):
    w = synth.WORKLOADS[name]
    s, d = w.edges(0, device=dev)
    g = G.granii_graph_csr_create(w.n, s, d, G.ADD_SELF_LOOPS | (G.SYMMETRIZE if w.symmetrize else 0))
    del s, d
    dinv = G.granii_graph_dinv(g)
    out = torch.empty(g.nnz, device=dev)
    f = lambda: G.granii_sddmm(g, G.SDDMM_DOT, dinv, 1, dinv, 1, 1, 1.0, out)
    f(); torch.cuda.synchronize()
    a, b = torch.cuda.Event(True), torch.cuda.Event(True)
    a.record()
    for _ in range(20): f()
    b.record(); torch.cuda.synchronize()
    ms = a.elapsed_time(b) / 20
    print(sys.argv[1] if len(sys.argv) > 1 else "", name, f"{ms:.4f} ms", f"{g.nnz * 12 / ms / 1e6:.0f} GB/s (12 B/entry)", flush=True)
    del g, out
    torch.cuda.empty_cache()
