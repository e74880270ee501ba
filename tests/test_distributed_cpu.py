"""Multi-process (gloo, world_size 2 and 3) CPU tests of the row-partitioned path.

What is checked here without a GPU:
  * the library's host partition (granii_partition_bounds) and gather-layout map
    (granii_gather_layout_host) on every rank, bit-exact against the oracle (O2);
  * the distributed data flow the CUDA layer implements (layer.cu): for every GCN
    composition, which dense operand is produced locally, padded into this rank's
    block and all-gathered, then aggregated over the local rows with remapped
    column ids; and the backward's all-gather + dW all-reduce.  Local compute is the
    fp64 oracle; the concatenation over ranks must equal the single-process oracle.
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import oracle as O
from paper_conf_cgo_lenadorasgytm26_b200 import synth


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _gather_rows(block, max_rows, world):
    """all-gather a [rows, K] block padded to max_rows -> [world*max_rows, K] (gather layout)"""
    pad = np.zeros((max_rows, block.shape[1]))
    pad[: block.shape[0]] = block
    t = torch.from_numpy(pad)
    out = [torch.zeros_like(t) for _ in range(world)]
    dist.all_gather(out, t)
    return torch.cat(out).numpy()


def _worker(rank, world, port, comps, ret):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from paper_conf_cgo_lenadorasgytm26_b200 import build
        build.build()
        from paper_conf_cgo_lenadorasgytm26_b200 import granii as G
        n, K1, K2 = 301, 13, 7
        s, d = synth.chung_lu(n, 1500, 2.4, seed=11)
        rp, ci = O.csr_build(n, s, d, O.SYMMETRIZE | O.ADD_SELF_LOOPS)
        bounds = G.granii_partition_bounds(rp, world)
        assert np.array_equal(bounds, O.partition(rp, world))
        max_rows = int(np.diff(bounds).max())
        b0, b1 = int(bounds[rank]), int(bounds[rank + 1])
        rp_loc = rp[b0:b1 + 1] - rp[b0]
        ci_glob = ci[rp[b0]:rp[b1]]
        ci_lay = G.granii_gather_layout_host(ci_glob, bounds, world, max_rows)
        # the layout map is a bijection back to global ids
        owner = ci_lay // max_rows
        assert np.array_equal(bounds[owner] + ci_lay - owner * max_rows, ci_glob)
        dinv = O.dinv(rp)
        dinv_lay = np.zeros(world * max_rows)
        for g in range(world):
            dinv_lay[g * max_rows: g * max_rows + bounds[g + 1] - bounds[g]] = dinv[bounds[g]:bounds[g + 1]]
        H = synth.features(1, n, K1).numpy().astype(np.float64)
        W = synth.glorot(2, 0, K1, K2, (K1, K2)).numpy().astype(np.float64)
        Gup = synth.uniform_pm1(3, 1, (n, K2)).numpy().astype(np.float64)
        Hl, dl = H[b0:b1], dinv[b0:b1]
        rows = np.repeat(np.arange(b1 - b0), np.diff(rp_loc))
        nval = dl[rows] * dinv_lay[ci_lay]                       # Ñ entries of the owned rows
        res = {}
        for comp in comps:
            if comp in (O.GCN_PRE_UPD, O.GCN_DYN_UPD):            # GEMM -> gather(T) -> SpMM
                T = O.gemm(Hl, W)
                if comp == O.GCN_DYN_UPD:
                    T = dl[:, None] * T                           # row-broadcast fused in the GEMM
                Tg = _gather_rows(T, max_rows, world)
                if comp == O.GCN_PRE_UPD:
                    Y = O.spmm(rp_loc, ci_lay, nval, Tg)
                else:
                    Y = dl[:, None] * O.spmm(rp_loc, ci_lay, None, Tg)
                S = None
            else:                                                 # gather(H) -> SpMM -> GEMM
                Hg = _gather_rows(Hl, max_rows, world)
                if comp == O.GCN_PRE_AGG:
                    S = O.spmm(rp_loc, ci_lay, nval, Hg)
                else:
                    S = dl[:, None] * O.spmm(rp_loc, ci_lay, None, dinv_lay[:, None] * Hg)
                Y = O.gemm(S, W)
            out = np.maximum(Y, 0)
            # backward: dY local, exchange per composition, dW all-reduced
            dY = np.where(Y > 0, Gup[b0:b1], 0.0)
            if comp in (O.GCN_PRE_UPD, O.GCN_DYN_UPD):
                dYg = _gather_rows(dY, max_rows, world)
                if comp == O.GCN_PRE_UPD:
                    dT = O.spmm(rp_loc, ci_lay, nval, dYg)        # Ñᵀ = Ñ (symmetric)
                else:
                    dT = dl[:, None] * O.spmm(rp_loc, ci_lay, None, dinv_lay[:, None] * dYg)
                dW = O.gemm(Hl, dT, ta=True)
                dH = O.gemm(dT, W, tb=True)
            else:
                dW = O.gemm(S, dY, ta=True)
                dS = O.gemm(dY, W, tb=True)
                if comp == O.GCN_DYN_AGG:
                    dS = dl[:, None] * dS
                dSg = _gather_rows(dS, max_rows, world)
                if comp == O.GCN_PRE_AGG:
                    dH = O.spmm(rp_loc, ci_lay, nval, dSg)
                else:
                    dH = dl[:, None] * O.spmm(rp_loc, ci_lay, None, dSg)
            t = torch.from_numpy(dW.copy())
            dist.all_reduce(t)
            res[comp] = (out, dH, t.numpy())
        ret[rank] = {"bounds": (b0, b1), "res": res}
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_row_partitioned_layer_matches_single_process(world):
    comps = list(O.GCN_COMPS)
    port = _free_port()
    manager = mp.Manager()
    ret = manager.dict()
    mp.start_processes(_worker, args=(world, port, comps, ret), nprocs=world, join=True, start_method="spawn")
    n, K1, K2 = 301, 13, 7
    s, d = synth.chung_lu(n, 1500, 2.4, seed=11)
    rp, ci = O.csr_build(n, s, d, O.SYMMETRIZE | O.ADD_SELF_LOOPS)
    H = synth.features(1, n, K1)
    W = synth.glorot(2, 0, K1, K2, (K1, K2))
    Gup = synth.uniform_pm1(3, 1, (n, K2))
    for comp in comps:
        ref, _ = O.gcn_forward(comp, rp, ci, H, W, 1)
        rdH, rdW = O.gcn_backward(comp, rp, ci, H, W, Gup, 1)
        out = np.concatenate([ret[r]["res"][comp][0] for r in range(world)])
        dH = np.concatenate([ret[r]["res"][comp][1] for r in range(world)])
        assert np.allclose(out, ref, rtol=1e-12, atol=1e-12)
        assert np.allclose(dH, rdH, rtol=1e-11, atol=1e-12)
        for r in range(world):
            assert np.allclose(ret[r]["res"][comp][2], rdW, rtol=1e-11, atol=1e-12)
