"""GAT scores + row softmax SDDMM (K = 1 ADD | LEAKYRELU | ROW_SOFTMAX, Eq. 4) timing on the workload
graphs, per shared-memory staging capacity (GRANII_SDDMM_CAP, read per launch): one line per
(graph, cap).  algorithmic bytes = per entry 4 B column + 4 B er + 4 B alpha, per row 16 B range + 4 B el."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
from paper_conf_cgo_lenadorasgytm26_b200 import granii as G, synth  # noqa: E402

dev = torch.device("cuda:0")
caps = sys.argv[1].split(",") if len(sys.argv) > 1 else ["0", "1024"]
graphs = sys.argv[2].split(",") if len(sys.argv) > 2 else ["pubmed", "arxiv", "reddit", "products"]
for name in graphs:
    w = synth.WORKLOADS[name]
    s, d = w.edges(0, device=dev)
    g = G.granii_graph_csr_create(w.n, s, d, G.ADD_SELF_LOOPS | (G.SYMMETRIZE if w.symmetrize else 0))
    del s, d
    el = synth.uniform_pm1(3, 1, (w.n,), device=dev)
    er = synth.uniform_pm1(3, 2, (w.n,), device=dev)
    out = torch.empty(g.nnz, device=dev)
    op = G.SDDMM_ADD | G.SDDMM_LEAKYRELU | G.SDDMM_ROW_SOFTMAX
    for cap in caps:
        os.environ["GRANII_SDDMM_CAP"] = cap
        f = lambda: G.granii_sddmm(g, op, el, 1, er, 1, 1, 1.0, out)
        f()
        torch.cuda.synchronize()
        a, b = torch.cuda.Event(True), torch.cuda.Event(True)
        a.record()
        for _ in range(20):
            f()
        b.record()
        torch.cuda.synchronize()
        ms = a.elapsed_time(b) / 20
        alg = g.nnz * 12 + w.n * 20
        print(f"{name} cap={cap} {ms:.4f} ms  {alg / ms / 1e6:.0f} GB/s algorithmic ({g.nnz} entries)", flush=True)
    del g, out
    torch.cuda.empty_cache()
