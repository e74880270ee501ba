"""Normwise error of every GAT backward output against the fp64 oracle on the parity-test cases
(diagnostic for the R22 tolerance): prints one line per (case, composition)."""
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))
import oracle as O  # noqa: E402
from paper_conf_cgo_lenadorasgytm26_b200 import granii as G, synth  # noqa: E402
import test_gpu_parity as T  # noqa: E402

CASES = [("pubmed", 32, 256, 1), ("pubmed", 64, 128, 0), ("dense", 48, 16, 1), ("sparse", 128, 47, 1),
         ("dense", 256, 1024, 0), ("dense", 384, 512, 0), ("directed_t", 64, 128, 0), ("directed_dense_t", 256, 64, 1)]
worst = {}
for name, K1, K2, act in CASES:
    c = T.case(G, name)
    for comp in (16, 17):
        net, out, H, W, al, ar = T.run_layer(G, c, G.GAT, comp, K1, K2, act, aligned=(K1 % 4 == 0))
        Gup = synth.uniform_pm1(61, 1, (c.n, K2))
        if act:
            Y, _ = O.gat_forward(comp, c.rp, c.ci, H, W, al, ar, 0)
            Gup[torch.from_numpy(np.abs(Y) < 1e-4 * np.abs(Y).max())] = 0.0
        dH = net.backward(T.pad(Gup), need_input_grad=True)
        torch.cuda.synchronize()
        ref = O.gat_backward(comp, c.rp, c.ci, H, W, al, ar, Gup, act)
        got = (dH, net.dW[0], net.da[0][0], net.da[0][1])
        errs = {nm: T.normwise(y.cpu(), r) for nm, y, r in zip(("dH", "dW", "da_l", "da_r"), got, ref)}
        for k, v in errs.items():
            worst[k] = max(worst.get(k, 0.0), v)
        print(name, K1, K2, act, G.COMP_NAMES[comp], " ".join(f"{k}={v:.2e}" for k, v in errs.items()), flush=True)
print("worst", " ".join(f"{k}={v:.2e}" for k, v in worst.items()))
