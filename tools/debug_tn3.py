import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
from paper_conf_cgo_lenadorasgytm26_b200 import granii as G
dev = torch.device('cuda:0')
rng = np.random.default_rng(0)
R, M, N = 64, 128, 32
A = rng.uniform(-1, 1, (R, M)); B = rng.uniform(-1, 1, (R, N))
Ad = torch.tensor(A, dtype=torch.float32, device=dev); Bd = torch.tensor(B, dtype=torch.float32, device=dev)
C = torch.zeros(M, N, device=dev)
print("ws bytes", G.granii_gemm_workspace_size(M, N, R, G.GEMM_TRANS_A))
ws = torch.full((G.granii_gemm_workspace_size(M, N, R, G.GEMM_TRANS_A) // 4,), 7.0, device=dev)
G.granii_profile_enable(True)
G.granii_gemm(M, N, R, Ad, M, Bd, N, C, N, G.GEMM_TRANS_A, workspace=ws.view(torch.uint8))
torch.cuda.synchronize()
print(G.granii_profile_read())
print("C", C[:2, :4].cpu().numpy(), "ws head", ws[:8].cpu().numpy())
print("ref", (A.T @ B)[:2, :4])
