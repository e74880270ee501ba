"""SpMM micro-sweep on the Reddit-shaped graph: time granii_spmm per (K, tune, slice) setting."""
import sys, os, json, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_cgo_lenadorasgytm26_b200 import granii as G, synth
from paper_conf_cgo_lenadorasgytm26_b200.model import alloc2d
dev = torch.device("cuda:0")
wname = sys.argv[1] if len(sys.argv) > 1 else "reddit"
w = synth.WORKLOADS[wname]
s, d = w.edges(0, device=dev)
g = G.granii_graph_csr_create(w.n, s, d, G.ADD_SELF_LOOPS | (G.SYMMETRIZE if w.symmetrize else 0))
dinv = G.granii_graph_dinv(g)
print("nnz", g.nnz, flush=True)
def t(K, reps=5):
    X = alloc2d(w.n, K, dev, fill=0.5); Y = alloc2d(w.n, K, dev)
    G.granii_spmm(g, None, X, K, Y, dinv, None, 0)
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(True), torch.cuda.Event(True)
    a.record()
    for _ in range(reps): G.granii_spmm(g, None, X, K, Y, dinv, None, 0)
    b.record(); torch.cuda.synchronize()
    ms = a.elapsed_time(b) / reps
    return ms, g.nnz * K * 4 / ms / 1e9
res = {}
for K in [int(x) for x in os.environ.get("KS", "256,41,64,128,1024").split(",")]:
    for tune in os.environ.get("TUNES", "def;2,4;4,4;4,2;8,2").split(";"):
        tune = "" if tune == "def" else tune
        for sl in os.environ.get("SLICES", "auto;64;128;256").split(";"):
            sl = "" if sl == "auto" else sl
            if sl and int(sl) >= K: continue
            os.environ.pop("GRANII_SPMM_TUNE", None); os.environ.pop("GRANII_SPMM_SLICE", None)
            if tune: os.environ["GRANII_SPMM_TUNE"] = tune
            if sl: os.environ["GRANII_SPMM_SLICE"] = sl
            ms, gbs = t(K)
            res[f"K{K} tune={tune or 'def'} slice={sl or 'auto'}"] = (round(ms, 3), round(gbs))
            print(f"K={K:5d} tune={tune or 'def':5s} slice={sl or 'auto':5s} {ms:8.3f} ms  {gbs:8.0f} GB/s gathered", flush=True)
