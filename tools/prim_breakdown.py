"""Per-primitive predicted vs measured time of single-layer compositions (selector diagnostics).

Measured: the library's tracer (granii_profile_*) over 5 forward calls of each composition.
Predicted: the calibrated per-primitive models, evaluated in Python from the same feature vectors
the C++ selector uses (granii_cost_features) and the coefficients of calib/b200.txt.
    python tools/prim_breakdown.py arxiv gat 256 512  [more "graph model K1 K2" groups ...]
"""
import json
import os
import sys

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_cgo_lenadorasgytm26_b200 import granii as G, synth  # noqa: E402
from paper_conf_cgo_lenadorasgytm26_b200.model import DEFAULT_CALIB, GNN, alloc2d  # noqa: E402
from regret_sweep import MODELS, spec_for  # noqa: E402

DEV = torch.device("cuda:0")


def coefs():
    c = {}
    for line in open(DEFAULT_CALIB):
        if line.startswith("#") or not line.strip():
            continue
        f = line.split()
        c[f[0]] = [float(x) for x in f[1:]]
    return c


def pred(g, C, prim, k1, k2=0):
    model, f = G.granii_cost_features(g, prim, k1, k2)
    return sum(a * b for a, b in zip(C[model], f)), model


def main(args):
    C = coefs()
    out = []
    for i in range(0, len(args), 4):
        name, mname, k1, k2 = args[i], args[i + 1], int(args[i + 2]), int(args[i + 3])
        w = synth.WORKLOADS[name]
        s, d = w.edges(0, DEV)
        g = G.granii_graph_csr_create(w.n, s, d, G.ADD_SELF_LOOPS | (G.SYMMETRIZE if w.symmetrize else 0))
        model = MODELS[mname]
        H = alloc2d(w.n, k1, DEV)
        H.copy_(synth.features(1, w.n, k1, device=DEV))
        _, comp_pred = G.granii_select_ex(g, model, G.shape_args(k1, k2, hops=2, Kh=k2 if model == G.GIN else 0),
                                          DEFAULT_CALIB, G.SELECT_NO_PREFILTER)
        for c in G.COMPS[model]:
            net = GNN(g, [spec_for(G, __import__("paper_conf_cgo_lenadorasgytm26_b200.model", fromlist=["LayerSpec"])
                                   .LayerSpec, model, k1, k2, c)], DEV)
            for _ in range(3):
                net.forward(H)
            torch.cuda.synchronize()
            G.granii_profile_enable(True)
            for _ in range(5):
                net.forward(H)
            prof = G.granii_profile_read()
            G.granii_profile_enable(False)
            meas = {k: v["ms"] / 5 for k, v in prof.items()}
            row = {"graph": name, "model": mname, "K1": k1, "K2": k2, "comp": G.COMP_NAMES[c],
                   "measured_ms": meas, "measured_total": sum(meas.values()),
                   "predicted_total": comp_pred.get(c)}
            # per-primitive predictions of the pieces a forward can contain
            pp = {}
            for pn, prim, a, b in (("spmm_w K1", G.P_SPMM_W, k1, 0), ("spmm_w K2", G.P_SPMM_W, k2, 0),
                                   ("spmm_u K1", G.P_SPMM_U, k1, 0), ("spmm_u K2", G.P_SPMM_U, k2, 0),
                                   ("spmm_u_cs K1", G.P_SPMM_U_CS, k1, 0), ("spmm_u_cs K2", G.P_SPMM_U_CS, k2, 0),
                                   ("sddmm1", G.P_SDDMM1, 0, 0), ("sddmm1_sm", G.P_SDDMM1_SM, 0, 0),
                                   ("gemm", G.P_GEMM, k1, k2), ("gemm_att", G.P_GEMM_ATT, k1, k2),
                                   ("gemm_nostore", G.P_GEMM_NOSTORE, k1, k2)):
                pp[pn] = round(pred(g, C, prim, a, b)[0], 4)
            row["primitive_predictions_ms"] = pp
            out.append(row)
            print(json.dumps(row), flush=True)
            del net
        del g, H
        torch.cuda.empty_cache()
    return out


if __name__ == "__main__":
    main(sys.argv[1:])
