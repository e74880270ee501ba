#!/usr/bin/env python
"""Selector regret over every BASELINE config graph plus the paper's Table II extremes
(SURVEY §8(d) R1 belgium_osm-like road graph, R2 mycielskian17-like dense graph).

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
    "pubmed": ("gcn", [(32, 32), (32, 256), (256, 32), (256, 256)]),
    "arxiv": ("gat", [(64, 128), (64, 256), (64, 512), (128, 256), (128, 512), (256, 512)]),
    "reddit": ("gcn", [(602, 32), (602, 256), (602, 1024), (256, 41), (1024, 41), (32, 256)]),
    "products": ("gcn+gat", [(100, 32), (100, 256), (100, 1024), (256, 47), (32, 256)]),
    "belgium": ("gcn", [(32, 32), (32, 256), (256, 32), (256, 256), (1024, 32), (32, 1024)]),
    "mycielskian": ("gcn", [(32, 32), (32, 256), (256, 32), (256, 256), (1024, 32), (32, 1024)]),
}


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


def main():
    out = {"device": torch.cuda.get_device_name(0), "calib": DEFAULT_CALIB, "when": time.strftime("%Y-%m-%d %H:%M"),
           "rows": []}
    calib = DEFAULT_CALIB if os.path.exists(DEFAULT_CALIB) else None
    for name, (models, pairs) in SWEEP.items():
        w = synth.WORKLOADS[name]
        s, d = w.edges(0, DEV)
        g = G.granii_graph_csr_create(w.n, s, d, G.ADD_SELF_LOOPS | (G.SYMMETRIZE if w.symmetrize else 0))
        print(f"[{name}] n={w.n} nnz={g.nnz}", flush=True)
        for mname in models.split("+"):
            model = G.GCN if mname == "gcn" else G.GAT
            comps = G.GCN_COMPS if model == G.GCN else G.GAT_COMPS
            for (k1, k2) in pairs:
                if model == G.GAT and k1 >= k2:
                    continue   # L330: GAT evaluated for increasing sizes only
                H = alloc2d(w.n, k1, DEV)
                H.copy_(synth.features(1, w.n, k1, device=DEV))
                W = synth.glorot(2, 0, k1, k2, (k1, k2), device=DEV).contiguous()
                al = synth.uniform_pm1(3, 0, (k2,), device=DEV)
                ar = synth.uniform_pm1(3, 1, (k2,), device=DEV)
                times = {}
                for c in comps:
                    net = GNN(g, [LayerSpec(model, k1, k2, G.ACT_RELU, comp=c, W=W, a_l=al, a_r=ar)], DEV)
                    times[G.COMP_NAMES[c]] = timeit(lambda: net.forward(H))
                    del net
                sel, pred = G.granii_select(g, model, k1, k2, calib)
                sel_np, _ = G.granii_select(g, model, k1, k2, calib, G.SELECT_NO_PREFILTER)
                best = min(times, key=times.get)
                if model == G.GCN:
                    cfg, static = ("GCN_DYN_UPD" if k1 > k2 else "GCN_DYN_AGG"), "GCN_DYN_AGG"
                else:
                    cfg, static = ("GAT_RECOMP" if k1 < k2 else "GAT_REUSE"), "GAT_REUSE"
                row = {"graph": name, "model": mname, "K1": k1, "K2": k2, "ms": times, "best": best,
                       "selected": G.COMP_NAMES[sel], "regret": times[G.COMP_NAMES[sel]] / times[best] - 1,
                       "regret_no_prefilter": times[G.COMP_NAMES[sel_np]] / times[best] - 1,
                       "config_regret": times[cfg] / times[best] - 1, "static_regret": times[static] / times[best] - 1,
                       "predicted_ms": {G.COMP_NAMES[k]: v for k, v in pred.items()}}
                out["rows"].append(row)
                print(f"  {mname} {k1:5d}->{k2:5d} best={best:12s} sel={row['selected']:12s} regret={row['regret']:.3f} "
                      f"config={row['config_regret']:.3f} static={row['static_regret']:.3f}", flush=True)
                del H
        del g
        torch.cuda.empty_cache()
    rg = [r["regret"] for r in out["rows"]]
    out["summary"] = {"n": len(rg), "max_regret": max(rg), "mean_regret": sum(rg) / len(rg),
                      "within_10pct": sum(x <= 0.10 for x in rg),
                      "max_config_regret": max(r["config_regret"] for r in out["rows"]),
                      "max_static_regret": max(r["static_regret"] for r in out["rows"])}
    print(json.dumps(out["summary"]))
    path = sys.argv[1] if len(sys.argv) > 1 else "gpurun_out/regret_sweep.json"
    json.dump(out, open(path, "w"), indent=1)


if __name__ == "__main__":
    main()
