import sys, os, subprocess
combos = ["4096,512,1024,3,1,4", "4096,1024,1024,3,1,4", "4096,512,512,3,1,4", "4096,256,1024,3,1,4", "512,4096,1024,3,1,4", "1024,4096,1024,3,1,4", "4096,512,1024,3,2,3", "4096,512,1024,0,2,3"]
for c in combos:
    env = dict(os.environ, GRANII_TN_DESC=c)
    out = subprocess.run([sys.executable, "-c", """
import sys; sys.path.insert(0, '.')
import numpy as np, torch
from paper_conf_cgo_lenadorasgytm26_b200 import granii as G
dev = torch.device('cuda:0')
rng = np.random.default_rng(0)
for (R, M, N) in [(32, 128, 32), (64, 128, 64)]:
    A = rng.uniform(-1, 1, (R, M)); B = rng.uniform(-1, 1, (R, N))
    Ad = torch.tensor(A, dtype=torch.float32, device=dev); Bd = torch.tensor(B, dtype=torch.float32, device=dev)
    C = torch.zeros(M, N, device=dev)
    G.granii_gemm(M, N, R, Ad, M, Bd, N, C, N, G.GEMM_TRANS_A); torch.cuda.synchronize()
    ref = A.T @ B; c = C.cpu().numpy()
    print('%.2e' % (np.abs(c - ref).max() / np.abs(ref).max()), '%.2e' % np.abs(c).max(), end=' | ')
"""], env=env, capture_output=True, text=True, timeout=120)
    print(c, "->", out.stdout.strip(), out.stderr.strip()[-200:])
