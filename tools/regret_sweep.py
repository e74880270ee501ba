#!/usr/bin/env python
"""Selector regret over every BASELINE config graph plus the paper's Table II extremes
(SURVEY §8(d) R1 belgium_osm-like road graph, R2 mycielskian17-like dense graph), for
GCN and GAT and the N3 models (SGC, TAGCN with k = 2 hops, GIN with Kh = K2).

For each (graph, K1, K2) every candidate composition of a single layer is timed
(forward; CUDA events, best of 3 x 5 repetitions) and compared with granii_select's
choice, the Config heuristic (L305 / Table VI: update-first iff K1 > K2 with DGL's
dynamic normalisation, L355; GAT: WiseGraph recomputes for growing sizes, L357) and
the static default (DYN_AGG / REUSE).  Writes one JSON file.
"""
import json
import os
import sys
import time

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_cgo_lenadorasgytm26_b200 import granii as G, synth  # noqa: E402
from paper_conf_cgo_lenadorasgytm26_b200.model import DEFAULT_CALIB, GNN, LayerSpec, alloc2d  # noqa: E402

DEV = torch.device("cuda:0")
SWEEP = {
    "cora": ("gcn", [(1433, 16)]),
    "pubmed": ("gcn+sgc+tagcn+gin", [(32, 32), (32, 256), (256, 32), (256, 256)]),
    "arxiv": ("gat", [(64, 128), (64, 256), (64, 512), (128, 256), (128, 512), (256, 512)]),
    "reddit": ("gcn+sgc+tagcn+gin", [(602, 32), (602, 256), (602, 1024), (256, 41), (1024, 41), (32, 256)]),
    "products": ("gcn+gat", [(100, 32), (100, 256), (100, 1024), (256, 47), (32, 256)]),
    "belgium": ("gcn+sgc+tagcn", [(32, 32), (32, 256), (256, 32), (256, 256), (1024, 32), (32, 1024)]),
    "mycielskian": ("gcn", [(32, 32), (32, 256), (256, 32), (256, 256), (1024, 32), (32, 1024)]),
}
MODELS = {"gcn": 0, "gat": 1, "sgc": 2, "tagcn": 3, "gin": 4}
# training (forward + backward of a hidden layer, dH included; SELECT_TRAINING costs the backward too)
TRAIN_SWEEP = {
    "pubmed": ("gcn+gat", [(32, 256), (256, 32), (64, 256)]),
    "arxiv": ("gcn+gat", [(128, 256), (256, 40), (64, 512)]),
    "reddit": ("gcn", [(602, 256), (256, 41), (32, 256)]),
    "products": ("gcn+gat", [(100, 256), (256, 47)]),
}


def spec_for(G, LayerSpec, model, k1, k2, comp=None):
    """one layer of each model; SGC / TAGCN with k = 2 hops, GIN with hidden width Kh = k2 (K2 = k2)"""
    W = synth.glorot(2, 0, k1, k2, (k1, k2), device=DEV).contiguous()
    if model == G.TAGCN:
        W = synth.glorot(2, 0, k1, k2, (3, k1, k2), device=DEV).contiguous()
    al = synth.uniform_pm1(3, 0, (k2,), device=DEV)
    ar = synth.uniform_pm1(3, 1, (k2,), device=DEV)
    W2 = synth.glorot(2, 1, k2, k2, (k2, k2), device=DEV).contiguous() if model == G.GIN else None
    return LayerSpec(model, k1, k2, G.ACT_RELU, comp=comp, W=W, a_l=al, a_r=ar, hops=2, eps=0.1,
                     Kh=k2 if model == G.GIN else 0, W2=W2)


def timeit(fn, reps=5, trials=3):
    best = 1e30
    for _ in range(trials):
        fn()
        torch.cuda.synchronize()
        a, b = torch.cuda.Event(True), torch.cuda.Event(True)
        a.record()
        for _ in range(reps):
            fn()
        b.record()
        torch.cuda.synchronize()
        best = min(best, a.elapsed_time(b) / reps)
    return best


def train_rows(out, calib):
    """fwd + bwd (hidden layer: dH computed) of every candidate vs SELECT_TRAINING's choice"""
    for name, (models, pairs) in TRAIN_SWEEP.items():
        w = synth.WORKLOADS[name]
        s, d = w.edges(0, DEV)
        fl = G.ADD_SELF_LOOPS | (G.SYMMETRIZE if w.symmetrize else G.BUILD_TRANSPOSE)
        g = G.granii_graph_csr_create(w.n, s, d, fl)
        print(f"[train {name}] n={w.n} nnz={g.nnz}", flush=True)
        for mname in models.split("+"):
            model = MODELS[mname]
            for (k1, k2) in pairs:
                H = alloc2d(w.n, k1, DEV)
                H.copy_(synth.features(1, w.n, k1, device=DEV))
                up = alloc2d(w.n, k2, DEV, fill=0.01)
                times = {}
                for c in G.COMPS[model]:
                    net = GNN(g, [spec_for(G, LayerSpec, model, k1, k2, c)], DEV)

                    def step():
                        net.forward(H)
                        net.backward(up, need_input_grad=True)
                    times[G.COMP_NAMES[c]] = timeit(step)
                    del net
                shape = G.shape_args(k1, k2)
                sel, pred = G.granii_select_ex(g, model, shape, calib, G.SELECT_TRAINING | G.SELECT_REFINE)
                sel_m, _ = G.granii_select_ex(g, model, shape, calib, G.SELECT_TRAINING)
                sel_np, pred_np = G.granii_select_ex(g, model, shape, calib, G.SELECT_TRAINING | G.SELECT_NO_PREFILTER)
                sel_f, _ = G.granii_select_ex(g, model, shape, calib)        # forward-only selection (the paper)
                best = min(times, key=times.get)
                row = {"graph": name, "model": mname, "mode": "fwd+bwd", "K1": k1, "K2": k2, "ms": times,
                       "best": best, "selected": G.COMP_NAMES[sel],
                       "regret": times[G.COMP_NAMES[sel]] / times[best] - 1,
                       "selected_model_only": G.COMP_NAMES[sel_m],
                       "regret_model_only": times[G.COMP_NAMES[sel_m]] / times[best] - 1,
                       "regret_no_prefilter": times[G.COMP_NAMES[sel_np]] / times[best] - 1,
                       "regret_forward_only_selection": times[G.COMP_NAMES[sel_f]] / times[best] - 1,
                       "config_regret": 0.0, "static_regret": 0.0,
                       "predicted_ms": {G.COMP_NAMES[k]: v for k, v in pred_np.items()}}
                row["pred_rel_err"] = {k: v / times[k] - 1 for k, v in row["predicted_ms"].items()}
                out["rows"].append(row)
                print(f"  train {mname} {k1:5d}->{k2:5d} best={best:12s} sel={row['selected']:12s} "
                      f"regret={row['regret']:.3f} model_only={row['regret_model_only']:.3f} "
                      f"fwd_sel={row['regret_forward_only_selection']:.3f}", flush=True)
                del H, up
        del g
        torch.cuda.empty_cache()


def main():
    out = {"device": torch.cuda.get_device_name(0), "calib": DEFAULT_CALIB, "when": time.strftime("%Y-%m-%d %H:%M"),
           "rows": []}
    calib = DEFAULT_CALIB if os.path.exists(DEFAULT_CALIB) else None
    train_only = "--train-only" in sys.argv
    for name, (models, pairs) in ({} if train_only else SWEEP).items():
        w = synth.WORKLOADS[name]
        s, d = w.edges(0, DEV)
        g = G.granii_graph_csr_create(w.n, s, d, G.ADD_SELF_LOOPS | (G.SYMMETRIZE if w.symmetrize else 0))
        print(f"[{name}] n={w.n} nnz={g.nnz}", flush=True)
        for mname in models.split("+"):
            model = MODELS[mname]
            comps = G.COMPS[model]
            for (k1, k2) in pairs:
                if model == G.GAT and k1 >= k2:
                    continue   # L330: GAT evaluated for increasing sizes only
                H = alloc2d(w.n, k1, DEV)
                H.copy_(synth.features(1, w.n, k1, device=DEV))
                times = {}
                for c in comps:
                    net = GNN(g, [spec_for(G, LayerSpec, model, k1, k2, c)], DEV)
                    times[G.COMP_NAMES[c]] = timeit(lambda: net.forward(H))
                    del net
                shape = G.shape_args(k1, k2, hops=2, Kh=k2 if model == G.GIN else 0)
                sel, pred = G.granii_select_ex(g, model, shape, calib, G.SELECT_REFINE)  # what GNN() runs
                sel_m, _ = G.granii_select_ex(g, model, shape, calib)                     # cost model alone
                sel_np, _ = G.granii_select_ex(g, model, shape, calib, G.SELECT_NO_PREFILTER)
                best = min(times, key=times.get)
                # Config heuristic (L305 / Table VI): update first iff K1 > K2 with DGL's dynamic
                # normalisation (L355); static = the framework default: aggregate first, dynamic
                # (DGL's GraphConv / SGConv / TAGConv / GINConv, L353), GAT reuse (L357)
                pre = mname.upper()
                if model == G.GAT:
                    cfg, static = ("GAT_RECOMP" if k1 < k2 else "GAT_REUSE"), "GAT_REUSE"
                else:
                    cfg, static = (f"{pre}_DYN_UPD" if k1 > k2 else f"{pre}_DYN_AGG"), f"{pre}_DYN_AGG"
                row = {"graph": name, "model": mname, "mode": "fwd", "K1": k1, "K2": k2, "ms": times, "best": best,
                       "selected": G.COMP_NAMES[sel], "regret": times[G.COMP_NAMES[sel]] / times[best] - 1,
                       "selected_model_only": G.COMP_NAMES[sel_m],
                       "regret_model_only": times[G.COMP_NAMES[sel_m]] / times[best] - 1,
                       "regret_no_prefilter": times[G.COMP_NAMES[sel_np]] / times[best] - 1,
                       "config_regret": times[cfg] / times[best] - 1, "static_regret": times[static] / times[best] - 1,
                       "predicted_ms": {G.COMP_NAMES[k]: v for k, v in pred.items()}}
                row["pred_rel_err"] = {k: v / times[k] - 1 for k, v in row["predicted_ms"].items()}
                out["rows"].append(row)
                print(f"  {mname} {k1:5d}->{k2:5d} best={best:12s} sel={row['selected']:12s} regret={row['regret']:.3f} "
                      f"config={row['config_regret']:.3f} static={row['static_regret']:.3f}", flush=True)
                del H
        del g
        torch.cuda.empty_cache()
    if "--no-train" not in sys.argv:
        train_rows(out, calib)
    rg = [r["regret"] for r in out["rows"]]
    out["summary"] = {"n": len(rg), "max_regret": max(rg), "mean_regret": sum(rg) / len(rg),
                      "within_10pct": sum(x <= 0.10 for x in rg),
                      "max_regret_model_only": max(r["regret_model_only"] for r in out["rows"]),
                      "within_10pct_model_only": sum(r["regret_model_only"] <= 0.10 for r in out["rows"]),
                      "max_config_regret": max(r["config_regret"] for r in out["rows"]),
                      "max_static_regret": max(r["static_regret"] for r in out["rows"])}
    for mode in ("fwd", "fwd+bwd"):
        rr = [r for r in out["rows"] if r["mode"] == mode]
        if rr:
            errs = sorted(abs(e) for r in rr for e in r["pred_rel_err"].values())
            out["summary_" + mode] = {"n": len(rr), "max_regret": max(r["regret"] for r in rr),
                                      "max_regret_model_only": max(r["regret_model_only"] for r in rr),
                                      "within_10pct_model_only": sum(r["regret_model_only"] <= 0.10 for r in rr),
                                      "pred_abs_rel_err_median": errs[len(errs) // 2], "pred_abs_rel_err_max": errs[-1]}
            print(mode, json.dumps(out["summary_" + mode]))
    out["summary_by_model"] = {}
    for mname in MODELS:
        rr = [r["regret"] for r in out["rows"] if r["model"] == mname]
        if rr:
            out["summary_by_model"][mname] = {"n": len(rr), "max_regret": max(rr), "mean_regret": sum(rr) / len(rr),
                                              "within_10pct": sum(x <= 0.10 for x in rr)}
    print(json.dumps(out["summary"]))
    print(json.dumps(out["summary_by_model"]))
    path = sys.argv[1] if len(sys.argv) > 1 else "gpurun_out/regret_sweep.json"
    json.dump(out, open(path, "w"), indent=1)


if __name__ == "__main__":
    main()
