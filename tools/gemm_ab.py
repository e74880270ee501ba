import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_cgo_lenadorasgytm26_b200 import granii as G
from paper_conf_cgo_lenadorasgytm26_b200.model import alloc2d
dev = torch.device("cuda:0")
R = 2449029
for (k1, k2, att) in [(100, 256, False), (100, 256, True), (256, 47, False), (256, 47, True), (602, 256, False)]:
    A = alloc2d(R, k1, dev, fill=0.5); W = torch.full((k1, k2), 0.01, device=dev); C = alloc2d(R, k2, dev)
    al = torch.full((k2,), 0.1, device=dev); ol = torch.empty(R, device=dev)
    ws = torch.empty(G.granii_gemm_workspace_size(R, k2, k1, 0), dtype=torch.uint8, device=dev)
    f = (lambda: G.granii_gemm(R, k2, k1, A, A.stride(0), W, k2, C, C.stride(0), 0, None, al, al, ol, ol, workspace=ws)) if att else \
        (lambda: G.granii_gemm(R, k2, k1, A, A.stride(0), W, k2, C, C.stride(0), workspace=ws))
    f(); torch.cuda.synchronize()
    a, b = torch.cuda.Event(True), torch.cuda.Event(True)
    best = 1e9
    for _ in range(3):
        a.record()
        for _ in range(10): f()
        b.record(); torch.cuda.synchronize(); best = min(best, a.elapsed_time(b) / 10)
    print(sys.argv[1], k1, k2, "att" if att else "   ", f"{best:.3f} ms", flush=True)
    del A, W, C, ws
