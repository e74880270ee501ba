import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
from paper_conf_cgo_lenadorasgytm26_b200 import granii as G
dev = torch.device("cuda:0")
np.set_printoptions(linewidth=200, precision=1, suppress=True)
def run(A, B):
    R, M = A.shape; N = B.shape[1]
    Ad = torch.tensor(A, dtype=torch.float32, device=dev); Bd = torch.tensor(B, dtype=torch.float32, device=dev)
    C = torch.zeros(M, N, device=dev)
    G.granii_gemm(M, N, R, Ad, M, Bd, N, C, N, G.GEMM_TRANS_A)
    torch.cuda.synchronize()
    return C.cpu().numpy()
R, M, N = 32, 128, 32
A = np.zeros((R, M)); 
for k in range(R): A[k, k] = 1.0          # C[m, n] = B[m, n] for m < 32
B = np.array([[k * 100 + n for n in range(N)] for k in range(R)], float)
C = run(A, B)
print("C[0:10, 0:6] (expect row m = 100m + n):"); print(C[0:10, 0:6])
print("C[30:34,0:4]"); print(C[30:34, 0:4])
# second probe: A all ones in column m=5 -> C[5, n] = sum_k B[k, n]
A2 = np.zeros((R, M)); A2[:, 5] = 1.0
C2 = run(A2, B)
print("row5 expect", B.sum(0)[:6], "got", C2[5, :6], "nonzero rows", np.nonzero(np.abs(C2).sum(1))[0][:10])
# random
rng = np.random.default_rng(0)
A3 = rng.uniform(-1, 1, (64, 128)); B3 = rng.uniform(-1, 1, (64, 32))
C3 = run(A3, B3); ref = A3.T @ B3
print("rand err", np.abs(C3 - ref).max() / np.abs(ref).max())
