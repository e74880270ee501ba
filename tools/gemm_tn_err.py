"""Accuracy and time of the dW GEMM C = Aᵀ·B (GRANII_GEMM_TRANS_A, tcgen05 3xTF32, split-K over the node
rows) against an fp64 product, as the reduction length R and the rows per split (GRANII_TN_SPLIT_ROWS,
read per call) vary: normwise max|C - ref| / max|ref| and ms per shape.  Diagnostic for the full-size
GAT / GCN dW tolerance (the reduction runs over every node row).
    python tools/gemm_tn_err.py [caps, e.g. 0,1024,2048] [R list]"""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_cgo_lenadorasgytm26_b200 import granii as G, synth  # noqa: E402
from paper_conf_cgo_lenadorasgytm26_b200.model import alloc2d  # noqa: E402

dev = torch.device("cuda:0")
caps = sys.argv[1].split(",") if len(sys.argv) > 1 else ["0"]
Rs = [int(x) for x in sys.argv[2].split(",")] if len(sys.argv) > 2 else [2500, 20000, 233000, 2449029]
shapes = [(256, 47), (100, 256), (602, 256)]


def run(M, N, R, A, B, C, cap):
    os.environ["GRANII_TN_SPLIT_ROWS"] = cap
    ws = torch.empty(G.granii_gemm_workspace_size(M, N, R, G.GEMM_TRANS_A), dtype=torch.uint8, device=dev)
    f = lambda: G.granii_gemm(M, N, R, A, A.stride(0), B, B.stride(0), C, N, G.GEMM_TRANS_A, workspace=ws)
    f()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(True), torch.cuda.Event(True)
    a.record()
    for _ in range(5):
        f()
    b.record()
    torch.cuda.synchronize()
    return a.elapsed_time(b) / 5


for R in Rs:
    for (M, N) in shapes:
        A = alloc2d(R, M, dev)
        A.copy_(synth.uniform_pm1(5, 1, (R, M), device=dev))
        B = alloc2d(R, N, dev)
        B.copy_(synth.uniform_pm1(5, 2, (R, N), device=dev))
        C = torch.empty((M, N), device=dev)
        ref = A.double().t() @ B.double()
        A2, B2 = alloc2d(R, M, dev), alloc2d(R, N, dev)   # positive (no cancellation: sums grow like R)
        A2.copy_(A.abs())
        B2.copy_(B.abs())
        ref2 = A2.double().t() @ B2.double()
        for cap in caps:
            ms = run(M, N, R, A, B, C, cap)
            nw = ((C.double() - ref).abs().max() / ref.abs().max()).item()
            run(M, N, R, A2, B2, C, cap)
            nw2 = ((C.double() - ref2).abs().max() / ref2.abs().max()).item()
            print(f"R={R} {M}x{N} cap={cap}: {ms:.4f} ms  normwise {nw:.2e} (random signs)  {nw2:.2e} (positive)",
                  flush=True)
        del A, B, C, ref, A2, B2, ref2
        torch.cuda.empty_cache()
