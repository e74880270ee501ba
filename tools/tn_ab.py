"""dW = A^T B (TN GEMM) timing for the Reddit / products shapes, GRANII_TN_BN = default / 128."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_cgo_lenadorasgytm26_b200 import granii as G
from paper_conf_cgo_lenadorasgytm26_b200.model import alloc2d
dev = torch.device("cuda:0")
for (R, M, N) in [(232965, 602, 256), (232965, 256, 41), (2449029, 100, 256), (232965, 602, 1024)]:
    A = alloc2d(R, M, dev, fill=0.5); B = alloc2d(R, N, dev, fill=0.25); C = torch.empty((M, N), device=dev)
    ws = torch.empty(G.granii_gemm_workspace_size(M, N, R, G.GEMM_TRANS_A), dtype=torch.uint8, device=dev)
    for mode in ("", "128", "", "128"):
        if mode: os.environ["GRANII_TN_BN"] = mode
        else: os.environ.pop("GRANII_TN_BN", None)
        f = lambda: G.granii_gemm(M, N, R, A, A.stride(0), B, B.stride(0), C, N, G.GEMM_TRANS_A, workspace=ws)
        f(); torch.cuda.synchronize()
        a, b = torch.cuda.Event(True), torch.cuda.Event(True)
        a.record()
        for _ in range(10): f()
        b.record(); torch.cuda.synchronize()
        print(R, M, N, mode or "def", f"{a.elapsed_time(b) / 10:.3f} ms", flush=True)
    del A, B, C, ws
