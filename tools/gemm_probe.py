import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_cgo_lenadorasgytm26_b200 import granii as G
from paper_conf_cgo_lenadorasgytm26_b200.model import alloc2d
dev = torch.device("cuda:0")
M = int(sys.argv[1]); K1 = int(sys.argv[2]); K2 = int(sys.argv[3])
A = alloc2d(M, K1, dev, fill=0.5); W = torch.full((K1, K2), 0.01, device=dev); C = alloc2d(M, K2, dev)
ws = torch.empty(G.granii_gemm_workspace_size(M, K2, K1, 0), dtype=torch.uint8, device=dev)
for _ in range(3): G.granii_gemm(M, K2, K1, A, A.stride(0), W, K2, C, C.stride(0), workspace=ws)
torch.cuda.synchronize()
a, b = torch.cuda.Event(True), torch.cuda.Event(True)
a.record()
for _ in range(10): G.granii_gemm(M, K2, K1, A, A.stride(0), W, K2, C, C.stride(0), workspace=ws)
b.record(); torch.cuda.synchronize()
ms = a.elapsed_time(b) / 10
print(f"M={M} {K1}->{K2}: {ms:.3f} ms, {(M*(K1+K2)*4)/ms/1e6:.0f} GB/s, {6*M*K1*K2/ms/1e9:.0f} TF/s (3xTF32-equiv)")
