"""Projected multi-GPU step time of a bench workload from ONE GPU (the pool has no 8-GPU box).

For G in --gpus, every rank r of the G-way row partition is built on this GPU in turn and
its step (forward [+ xent + backward + SGD]) is timed with CUDA events through a TIMING-STUB
communicator (granii_comm_create_stub: collectives move no data, they only count the bytes
this rank would receive).  So the per-rank compute is MEASURED -- including the block-phased
SpMM overhead of the overlapped path -- and the communication is MODELLED:

  t_comm        = bytes received per rank per step / bus bandwidth (--bw_gbs, assumed)
  no_overlap_ms = max_r t_compute(r) + t_comm
  overlap_ms    = max(max_r t_compute(r), t_comm)        (perfect overlap: the lower bound)

Both are reported with edges/s = stored entries x layers / time.  This is a projection, not
a multi-GPU measurement; bench.py under torchrun measures the real thing on a multi-GPU box.
"""
from __future__ import annotations

import argparse
import json
import os
import sys

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import bench  # noqa: E402
from paper_conf_cgo_lenadorasgytm26_b200 import synth  # noqa: E402


def rank_step_ms(G, spec, w, src, dst, flags, rank, world, dev, steps, warmup, comps=None):
    from paper_conf_cgo_lenadorasgytm26_b200.model import alloc2d
    comm = G.granii_comm_create_stub(rank, world) if world > 1 else None
    g = G.granii_graph_csr_create(w.n, src, dst, flags, rank, world)
    info = g.info
    R = g.n_rows
    dims = spec["dims"]
    H = alloc2d(R, dims[0], dev)
    H.copy_(synth.features(1, w.n, dims[0], device=dev)[info.row_begin:info.row_end])
    labels = synth.labels(4, w.n, dims[-1], device=dev)[info.row_begin:info.row_end].contiguous()
    net = bench.build_model(G, None, spec, g, dev, comm)
    if comps:
        for L, c in zip(net.layers, comps):
            L.comp = c
        net = type(net)(g, net.layers, dev, comm)
    dlogits = alloc2d(R, dims[-1], dev)
    loss = torch.zeros(max(R, 1), device=dev)

    def step():
        if spec["train"]:
            net.train_step(H, labels, w.n, 0.01, dlogits, loss)
        else:
            net.forward(H)

    for _ in range(warmup):
        step()
    torch.cuda.synchronize()
    b0 = G.granii_comm_stats(comm)[0] if comm else 0
    ms = bench.time_region(step, steps, torch.cuda.current_stream())
    b1 = G.granii_comm_stats(comm)[0] if comm else 0
    G.granii_profile_enable(True)   # per-primitive breakdown of one more step (not the timed ones)
    step()
    torch.cuda.synchronize()
    prof = {k: round(v["ms"], 4) for k, v in G.granii_profile_read().items()}
    G.granii_profile_enable(False)
    out = {"rank": rank, "rows": R, "local_nnz": info.local_nnz, "compute_ms": ms, "per_primitive_ms": prof,
           "bytes_in_per_step": (b1 - b0) / steps, "compositions": [L.comp for L in net.layers]}
    if world > 1:   # the planner's schedule for every aggregation width of the model (N1)
        out["plan"] = {}
        for K in sorted(set(dims)):
            for kind, wgt, cs in (("weighted", True, False), ("unweighted", False, False), ("col_scale", False, True)):
                P, t1, tp = G.granii_comm_plan(g, K, wgt, cs)
                out["plan"][f"K{K}_{kind}"] = {"phases": P, "model_ms_allgather_then_spmm": t1, "model_ms_planned": tp}
    del net, g, H
    torch.cuda.empty_cache()
    return out, info.nnz


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--workload", default="reddit-gcn2-train", choices=sorted(bench.WORKLOADS))
    ap.add_argument("--gpus", default="1,2,4,8")
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--bw_gbs", type=float, default=650.0,
                    help="assumed NCCL bus bandwidth per GPU on NVLink 5 (not measurable on a 1-GPU pool)")
    ap.add_argument("--overlap", default="1", choices=["0", "1"],
                    help="GRANII_COMM_OVERLAP: 1 = block-phased SpMM (default), 0 = all-gather then SpMM")
    ap.add_argument("--ranks", default=None, help="time only these ranks (e.g. 0,7)")
    ap.add_argument("--comp", default=None, help="force the compositions, e.g. 3,3 (skips the selector)")
    ap.add_argument("--out", default=None)
    args = ap.parse_args()
    os.environ["GRANII_COMM_OVERLAP"] = args.overlap
    from paper_conf_cgo_lenadorasgytm26_b200 import granii as G
    dev = torch.device("cuda", 0)
    torch.cuda.set_device(dev)
    spec = bench.WORKLOADS[args.workload]
    w = synth.WORKLOADS[spec["graph"]]
    src, dst = w.edges(seed=0, device=dev)
    flags = G.ADD_SELF_LOOPS | (G.SYMMETRIZE if w.symmetrize else 0)
    layers = len(spec["dims"]) - 1
    passes = spec.get("hops", 1) if spec["model"] in ("sgc", "tagcn") else 1
    res = {"workload": args.workload, "assumed_bus_gbs": args.bw_gbs, "kind": "projection",
           "how": __doc__.split("\n\n")[1].replace("\n", " "), "per_G": {}}
    for world in [int(x) for x in args.gpus.split(",")]:
        ranks = []
        sel = range(world) if not args.ranks else [int(x) for x in args.ranks.split(",") if int(x) < world]
        for r in sel:
            comps = [int(x) for x in args.comp.split(",")] if args.comp else None
            o, nnz = rank_step_ms(G, spec, w, src, dst, flags, r, world, dev, args.steps, args.warmup, comps)
            ranks.append(o)
            print(json.dumps({"G": world, **o}), flush=True)
        tc = max(o["compute_ms"] for o in ranks)
        world_n = len(ranks)
        bytes_in = max(o["bytes_in_per_step"] for o in ranks)
        tcomm = bytes_in / (args.bw_gbs * 1e9) * 1e3
        edges = float(nnz) * layers * passes
        res["per_G"][str(world)] = {
            "max_rank_compute_ms": tc, "mean_rank_compute_ms": sum(o["compute_ms"] for o in ranks) / world_n, "overlap": args.overlap,
            "bytes_in_per_rank_per_step": bytes_in, "modelled_comm_ms": tcomm,
            "no_overlap_ms": tc + tcomm, "overlap_bound_ms": max(tc, tcomm),
            "edges_per_s_no_overlap": edges / ((tc + tcomm) / 1e3),
            "edges_per_s_overlap_bound": edges / (max(tc, tcomm) / 1e3),
            "compositions": sorted({tuple(o["compositions"]) for o in ranks}), "ranks": ranks}
    base = res["per_G"].get("1")
    if base:
        for k, v in res["per_G"].items():
            v["speedup_no_overlap"] = base["no_overlap_ms"] / v["no_overlap_ms"]
            v["speedup_overlap_bound"] = base["no_overlap_ms"] / v["overlap_bound_ms"]
    s = json.dumps(res, indent=1, default=list)
    print(s)
    if args.out:
        open(args.out, "w").write(s)


if __name__ == "__main__":
    main()
