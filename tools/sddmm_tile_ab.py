"""K = 1 SDDMM A/B: entry tiles (GRANII_SDDMM_TILE=1) vs the degree-ordered kernel (0) on the workload
graphs, for the normalisation scores (DOT of D^-1/2, D^-1/2) and the GAT scores + row softmax (ADD |
LEAKYRELU | ROW_SOFTMAX, Eq. 4).  One line per (graph, op, variant): ms per launch (CUDA events, 20
launches) and GB/s of compulsory bytes (per entry 4 B column + 4 B output, per row 8 B row_ptr + 4 B U;
the V gather counted once per column), plus the max |difference| between the two variants."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
from paper_conf_cgo_lenadorasgytm26_b200 import granii as G, synth  # noqa: E402

dev = torch.device("cuda:0")
graphs = sys.argv[1].split(",") if len(sys.argv) > 1 else ["pubmed", "arxiv", "reddit", "products"]
variants = sys.argv[2].split(",") if len(sys.argv) > 2 else ["0", "1"]
ops = sys.argv[3].split(",") if len(sys.argv) > 3 else ["norm", "att"]
for name in graphs:
    w = synth.WORKLOADS[name]
    s, d = w.edges(0, device=dev)
    g = G.granii_graph_csr_create(w.n, s, d, G.ADD_SELF_LOOPS | (G.SYMMETRIZE if w.symmetrize else 0))
    del s, d
    dinv = G.granii_graph_dinv(g)
    el = synth.uniform_pm1(3, 1, (w.n,), device=dev)
    er = synth.uniform_pm1(3, 2, (w.n,), device=dev)
    comp = g.nnz * 8 + w.n * 16
    for opname, op, U, V in (("norm", G.SDDMM_DOT, dinv, dinv),
                             ("att", G.SDDMM_ADD | G.SDDMM_LEAKYRELU | G.SDDMM_ROW_SOFTMAX, el, er)):
        if opname not in ops:
            continue
        outs = {}
        for tile in variants:
            os.environ["GRANII_SDDMM_TILE"] = tile
            out = torch.empty(g.nnz, device=dev)
            f = lambda: G.granii_sddmm(g, op, U, 1, V, 1, 1, 1.0, out)
            f()
            torch.cuda.synchronize()
            a, b = torch.cuda.Event(True), torch.cuda.Event(True)
            a.record()
            for _ in range(20):
                f()
            b.record()
            torch.cuda.synchronize()
            ms = a.elapsed_time(b) / 20
            outs[tile] = out
            print(f"{name} {opname} tile={tile} {ms:.4f} ms  {comp / ms / 1e6:.0f} GB/s compulsory ({g.nnz} entries)",
                  flush=True)
        if len(outs) == 2:
            print(f"{name} {opname} max|tile - ordered| = {(outs['0'] - outs['1']).abs().max().item():.3e}", flush=True)
        del outs
    del g
    torch.cuda.empty_cache()
