#!/usr/bin/env python
"""B200 calibration of GRANII's per-primitive cost models (§IV-E;
the paper's "initialization script that gathers profiling data and trains its cost
models", L155).

Times every primitive through the C ABI on a sweep of synthetic graphs that is
DISJOINT from the benchmark / test workloads (other sizes, densities and seeds),
pairs each time with the feature vector the C++ selector uses
(granii_cost_features), and fits each model's coefficients by non-negative least
squares weighted by 1/t (relative error).  Writes calib/b200.txt.

    python tools/calibrate.py [--out calib/b200.txt] [--quick]
"""
from __future__ import annotations

import argparse
import json
import os
import sys
import time

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_cgo_lenadorasgytm26_b200 import granii as G, synth  # noqa: E402
from paper_conf_cgo_lenadorasgytm26_b200.model import alloc2d  # noqa: E402

DEV = torch.device("cuda:0")

# (name, generator, n, m, param, seed, symmetric) -- none equals a bench/test workload
GRAPHS = [
    ("cl-50k-sparse", "chung_lu", 50_000, 150_000, 2.5, 101, True),
    ("cl-300k-mid", "chung_lu", 300_000, 2_000_000, 2.3, 102, True),
    ("cl-100k-dense", "chung_lu", 100_000, 8_000_000, 2.2, 103, True),
    ("cl-600k-power", "chung_lu", 600_000, 20_000_000, 2.6, 104, True),
    ("cl-150k-vdense", "chung_lu", 150_000, 30_000_000, 3.5, 106, True),
    ("rmat-400k", "rmat", 400_000, 4_000_000, None, 107, False),
    ("rmat-1.5m", "rmat", 1_500_000, 15_000_000, None, 108, True),
    ("road-800k", "road", 800_000, 0, None, 109, True),
    ("rmat-200k-dir", "rmat", 200_000, 1_600_000, None, 110, False),
    ("rmat-3m", "rmat", 3_000_000, 40_000_000, None, 111, True),
    ("cl-250k-dense", "chung_lu", 250_000, 45_000_000, 2.8, 112, True),
    ("cl-30k", "chung_lu", 30_000, 120_000, 2.4, 113, True),
]
KS = [16, 32, 64, 128, 256, 512]
GEMM_PAIRS = [(32, 32), (64, 256), (256, 64), (100, 256), (602, 256), (256, 41), (1024, 128), (128, 1024),
              (512, 512), (1433, 16)]


def timed(fn, reps=3):
    fn()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(True), torch.cuda.Event(True)
    a.record()
    for _ in range(reps):
        fn()
    b.record()
    torch.cuda.synchronize()
    return a.elapsed_time(b) / reps


def make_graph(kind, n, m, p, seed, sym):
    if kind == "chung_lu":
        s, d = synth.chung_lu(n, m, p, seed, DEV, max_w_frac=0.002)
    elif kind == "rmat":
        s, d = synth.rmat(n, m, 0.57, 0.19, 0.19, seed, DEV)
    else:
        s, d = synth.road(n, seed, DEV)
    return G.granii_graph_csr_create(n, s, d, G.ADD_SELF_LOOPS | (G.SYMMETRIZE if sym else 0))


def sweep(quick=False):
    samples = []
    graphs = GRAPHS[:3] if quick else GRAPHS
    for (name, kind, n, m, p, seed, sym) in graphs:
        g = make_graph(kind, n, m, p, seed, sym)
        R = g.n_rows
        dinv = G.granii_graph_dinv(g)
        print(f"[{name}] rows={R} nnz={g.nnz}", flush=True)

        def rec(prim, K1, K2, ms):
            model, f = G.granii_cost_features(g, prim, K1, K2)
            samples.append({"graph": name, "prim": prim, "model": model, "K1": K1, "K2": K2, "f": f, "ms": ms})

        vals = torch.full((max(g.nnz, 1),), 0.25, device=DEV)
        for K in KS:
            X = alloc2d(R, K, DEV, fill=0.5)
            Y = alloc2d(R, K, DEV)
            rec(G.P_SPMM_W, K, 0, timed(lambda: G.granii_spmm(g, vals, X, K, Y)))
            rec(G.P_SPMM_U, K, 0, timed(lambda: G.granii_spmm(g, None, X, K, Y, dinv, None)))
            rec(G.P_SPMM_U_CS, K, 0, timed(lambda: G.granii_spmm(g, None, X, K, Y, dinv, dinv)))
            del X, Y
        out = torch.empty(max(g.nnz, 1), device=DEV)
        el = torch.full((R,), 0.1, device=DEV)
        rec(G.P_SDDMM1, 0, 0, timed(lambda: G.granii_sddmm(g, G.SDDMM_DOT, dinv, 1, dinv, 1, 1, 1.0, out)))
        rec(G.P_SDDMM1_SM, 0, 0, timed(lambda: G.granii_sddmm(
            g, G.SDDMM_ADD | G.SDDMM_LEAKYRELU | G.SDDMM_ROW_SOFTMAX, el, 1, el, 1, 1, 1.0, out)))
        if sym:  # GAT backward passes (symmetric graphs; per-pass times from the library's tracer)
            from paper_conf_cgo_lenadorasgytm26_b200.model import GNN, LayerSpec
            for K in KS:
                k1 = 16
                W = torch.full((k1, K), 0.01, device=DEV)
                av = torch.full((K,), 0.05, device=DEV)
                net = GNN(g, [LayerSpec(G.GAT, k1, K, G.ACT_RELU, comp=G.GAT_REUSE, W=W, a_l=av, a_r=av)], DEV)
                X = alloc2d(R, k1, DEV, fill=0.5)
                gup = alloc2d(R, K, DEV, fill=0.01)
                net.forward(X)
                net.backward(gup)
                torch.cuda.synchronize()
                G.granii_profile_enable(True)
                for _ in range(3):
                    net.backward(gup)
                torch.cuda.synchronize()
                prof = G.granii_profile_read()
                G.granii_profile_enable(False)
                rec(G.P_GAT_BWD_A, K, 0, prof["gat_bwd_a"]["ms"] / prof["gat_bwd_a"]["calls"])
                rec(G.P_GAT_BWD_B, K, 0, prof["gat_bwd_b"]["ms"] / prof["gat_bwd_b"]["calls"])
                del net, X, gup
            # the der-only pass of a RECOMP input layer (no dH): independent of K
            W = torch.full((64, 16), 0.01, device=DEV)
            av = torch.full((16,), 0.05, device=DEV)
            net = GNN(g, [LayerSpec(G.GAT, 64, 16, G.ACT_RELU, comp=G.GAT_RECOMP, W=W, a_l=av, a_r=av)], DEV)
            X = alloc2d(R, 64, DEV, fill=0.5)
            gup = alloc2d(R, 16, DEV, fill=0.01)
            net.forward(X)
            net.backward(gup, need_input_grad=False)
            torch.cuda.synchronize()
            G.granii_profile_enable(True)
            for _ in range(3):
                net.backward(gup, need_input_grad=False)
            torch.cuda.synchronize()
            prof = G.granii_profile_read()
            G.granii_profile_enable(False)
            rec(G.P_GAT_DER, 0, 0, prof["gat_der"]["ms"] / prof["gat_der"]["calls"])
            del net, X, gup
        for (k1, k2) in GEMM_PAIRS:
            A = alloc2d(R, k1, DEV, fill=0.5)
            W = torch.full((k1, k2), 0.01, device=DEV)
            C = alloc2d(R, k2, DEV)
            ws = torch.empty(G.granii_gemm_workspace_size(R, k2, k1, 0), dtype=torch.uint8, device=DEV)
            rec(G.P_GEMM, k1, k2, timed(lambda: G.granii_gemm(R, k2, k1, A, A.stride(0), W, k2, C, C.stride(0),
                                                               workspace=ws)))
            al = torch.full((k2,), 0.1, device=DEV)
            ol = torch.empty(R, device=DEV)
            ws2 = torch.empty(G.granii_gemm_workspace_size(R, k2, k1, G.GEMM_NO_STORE), dtype=torch.uint8, device=DEV)
            rec(G.P_GEMM_NOSTORE, k1, k2, timed(lambda: G.granii_gemm(
                R, k2, k1, A, A.stride(0), W, k2, None, k2, G.GEMM_NO_STORE, None, al, al, ol, ol, workspace=ws2)))
            rec(G.P_GEMM_ATT, k1, k2, timed(lambda: G.granii_gemm(
                R, k2, k1, A, A.stride(0), W, k2, C, C.stride(0), 0, None, al, al, ol, ol, workspace=ws2)))
            dW = torch.empty((k1, k2), device=DEV)
            ws3 = torch.empty(G.granii_gemm_workspace_size(k1, k2, R, G.GEMM_TRANS_A), dtype=torch.uint8, device=DEV)
            rec(G.P_GEMM_TN, k1, k2, timed(lambda: G.granii_gemm(k1, k2, R, A, A.stride(0), C, C.stride(0), dW, k2,
                                                                  G.GEMM_TRANS_A, workspace=ws3)))
            del A, C, ws, ws2, ws3
        del g
        torch.cuda.empty_cache()
    return samples


def fit(samples):
    from scipy.optimize import nnls
    coefs, report = {}, {}
    for model in sorted({s["model"] for s in samples}):
        S = [s for s in samples if s["model"] == model]
        F = np.array([s["f"] for s in S])
        y = np.array([s["ms"] for s in S])
        w = 1.0 / np.maximum(y, 1e-3)
        c, _ = nnls(F * w[:, None], y * w)
        pred = F @ c
        rel = np.abs(pred - y) / y
        coefs[model] = c
        report[model] = {"n": len(S), "median_rel_err": float(np.median(rel)), "max_rel_err": float(rel.max())}
    return coefs, report


GEMM_FEATS = {"gemm": 4, "gemm_att": 5, "gemm_tn": 4}  # feature counts before the roofline-time feature


def augment(samples):
    """samples measured before the GEMM models' roofline-time feature (select.cpp gemm_roof_ms): append
    max(HBM GB / 6.53, TFLOP x 3 / 0.705) computed from the sample's own HBM GB and TFLOP features"""
    for s in samples:
        n = GEMM_FEATS.get(s["model"])
        if n is not None and len(s["f"]) == n:
            s["f"] = list(s["f"]) + [max(s["f"][1] / 6.53, s["f"][2] * 3.0 / 0.705)]
    return samples


def relabel(samples):
    """model keys of samples taken before the warp-per-row / group-per-row split (select.cpp
    group_mode: average degree < 16): the graph's average degree from its K = 16 unweighted SpMM
    sample (streamed GB = nnz x 4 B for an unsliced SpMM, M rows)"""
    avg = {}
    for s in samples:
        if s["prim"] == 1 and s["K1"] == 16:
            avg[s["graph"]] = s["f"][1] / 4e-9 / (s["f"][5] * 1e6)
    for s in samples:
        if s["model"] in ("spmm", "gat_bwd_a", "gat_bwd_b") and avg.get(s["graph"], 99.0) < 16.0:
            s["model"] += "_g"
    return samples


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--out", default=os.path.join(ROOT, "calib", "b200.txt"))
    ap.add_argument("--quick", action="store_true")
    ap.add_argument("--refit", default=None, help="refit from a saved *_samples.json instead of measuring")
    args = ap.parse_args()
    t0 = time.time()
    samples = augment(relabel(json.load(open(args.refit))["samples"])) if args.refit else sweep(args.quick)
    coefs, report = fit(samples)
    os.makedirs(os.path.dirname(args.out), exist_ok=True)
    with open(args.out, "w") as f:
        f.write(f"# GRANII B200 cost-model coefficients (tools/calibrate.py, {len(samples)} samples, "
                f"{'refit of ' + args.refit if args.refit else torch.cuda.get_device_name(0)}, "
                f"{time.strftime('%Y-%m-%d')})\n")
        f.write("# model coef... (feature order: paper_conf_cgo_lenadorasgytm26_b200/csrc/select.cpp)\n")
        for model, c in coefs.items():
            f.write(f"# {model}: n={report[model]['n']} median rel err {report[model]['median_rel_err']:.3f} "
                    f"max {report[model]['max_rel_err']:.3f}\n")
            f.write(model + " " + " ".join(f"{x:.6g}" for x in c) + "\n")
    json.dump({"samples": samples, "report": report}, open(args.out.replace(".txt", "_samples.json"), "w"))
    print(json.dumps(report, indent=1))
    print(f"wrote {args.out} in {time.time() - t0:.0f} s")


if __name__ == "__main__":
    main()
