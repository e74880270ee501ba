import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import oracle as O
from paper_conf_cgo_lenadorasgytm26_b200 import granii as G, synth
from paper_conf_cgo_lenadorasgytm26_b200.model import alloc2d
dev = torch.device("cuda:0")
def run(M, N, K, exact=False):
    A = synth.uniform_pm1(1, 1, (M, K)); B = synth.uniform_pm1(1, 2, (K, N))
    if exact:  # values with 10-bit mantissa -> tf32-exact, lo == 0
        A = (A * 512).round() / 512; B = (B * 512).round() / 512
    Ad = alloc2d(M, K, dev); Ad.copy_(A); C = alloc2d(M, N, dev); C.zero_()
    G.granii_gemm(M, N, K, Ad, Ad.stride(0), B.to(dev).contiguous(), N, C, C.stride(0))
    torch.cuda.synchronize()
    r = O.gemm(A, B); c = C.cpu().numpy()
    return np.abs(c - r).max() / np.abs(r).max()
for N in (16, 256):
    for K in (32, 64, 96, 128, 160, 256):
        print(f"N={N} K={K} err={run(512, N, K):.2e} exact={run(512, N, K, True):.2e}", flush=True)
