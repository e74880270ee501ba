#!/usr/bin/env python
"""Dump one GAT backward case (GPU outputs + inputs) to gpurun_out/gat_bwd_<case>.npz for host analysis."""
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))
import test_gpu_parity as T  # noqa: E402
from paper_conf_cgo_lenadorasgytm26_b200 import granii as G, synth  # noqa: E402


def main(name="pubmed", comp=16, K1=32, K2=256, act=1):
    c = T.case(G, name)
    net, out, H, W, al, ar = T.run_layer(G, c, G.GAT, comp, K1, K2, act)
    Gup = synth.uniform_pm1(61, 1, (c.n, K2))
    dH = net.backward(T.pad(Gup), need_input_grad=True)
    torch.cuda.synchronize()
    os.makedirs("gpurun_out", exist_ok=True)
    # inputs are regenerated on the host from the same seeds (synth is device-independent)
    np.savez_compressed(f"gpurun_out/gat_bwd_{name}_{comp}_{act}.npz", dH=dH.cpu().numpy(),
                        dW=net.dW[0].cpu().numpy(), dal=net.da[0][0].cpu().numpy(), dar=net.da[0][1].cpu().numpy())


if __name__ == "__main__":
    a = sys.argv[1:]
    main(a[0], int(a[1]), int(a[2]), int(a[3]), int(a[4])) if a else main()
