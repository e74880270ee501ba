"""The row-partitioned path run on ONE GPU (-m gpu).

G ranks are host threads of this process, each on its own CUDA stream, joined by
the library's in-process loopback communicator (granii_comm_create_local): the
collectives are host barriers plus stream-ordered device copies, so every
device-side piece of the multi-GPU path runs here exactly as under NCCL -- the
nnz-balanced partition, gather-layout column ids, dinv of the gather layout,
producers writing into their slot of the padded all-gather buffer, the layer
compositions on owned rows, the block-phased SpMM that overlaps the per-block
broadcasts (N1; GRANII_COMM_OVERLAP=0 falls back to all-gather -> SpMM), and the
dW / da all-reduce.  The concatenation of the
ranks' owned rows must match the single-process fp64 oracle within the same
tolerances as the unpartitioned path (test_gpu_parity.py, R19 / R22).
"""
import os
import time
import threading

import numpy as np
import pytest
import torch

import oracle as O
from paper_conf_cgo_lenadorasgytm26_b200 import synth
from test_gpu_parity import TOL, err, err_act, gat_grad_ok

pytestmark = pytest.mark.gpu
DEV = torch.device("cuda:0") if torch.cuda.is_available() else None
F = O.ADD_SELF_LOOPS | O.SYMMETRIZE


@pytest.fixture(scope="module")
def G():
    from paper_conf_cgo_lenadorasgytm26_b200 import granii
    return granii


def graph_case(name):
    if name == "sparse":
        n = 2000
        s, d = synth.chung_lu(n, 5000, 2.5, seed=21)
    elif name == "dense":
        n = 1500
        s, d = synth.chung_lu(n, 60000, 2.1, seed=22, max_w_frac=0.05)
    else:
        n = 45
        s, d = synth.random_small(n, 120, 23)
    return n, s, d


def run_ranks(G, world, n, s, d, body, flags=F):
    """create the G partitioned graphs, then run body(rank, graph, comm, rows) on G threads;
    returns the per-rank results in rank order"""
    sd, dd = s.to(DEV).contiguous(), d.to(DEV).contiguous()
    graphs = [G.granii_graph_csr_create(n, sd, dd, flags, r, world) for r in range(world)]
    comms = G.granii_comm_create_local(world)
    res, errs = [None] * world, []

    def worker(r):
        try:
            torch.cuda.set_device(DEV)
            st = torch.cuda.Stream(DEV)
            with torch.cuda.stream(st):
                info = graphs[r].info
                res[r] = body(r, graphs[r], comms[r], (info.row_begin, info.row_end))
                st.synchronize()
        except BaseException as e:  # noqa: BLE001 -- re-raised in the main thread
            errs.append(e)

    th = [threading.Thread(target=worker, args=(r,)) for r in range(world)]
    for t in th:
        t.start()
    for t in th:
        t.join(timeout=300)
    assert not any(t.is_alive() for t in th), "rank thread hung (collective mismatch)"
    if errs:
        raise errs[0]
    torch.cuda.synchronize()
    return res, graphs


def padded(x):
    from paper_conf_cgo_lenadorasgytm26_b200.model import alloc2d
    x = torch.as_tensor(x, dtype=torch.float32)
    out = alloc2d(x.shape[0], x.shape[1], DEV)
    out.copy_(x)
    return out


@pytest.mark.parametrize("world", [2, 3, 4])
@pytest.mark.parametrize("name", ["sparse", "dense", "tiny"])
def test_partitioned_csr_concatenates_to_global(G, world, name):
    """O2: bounds bit-exact vs the oracle, the ranks' local CSRs concatenate to the global CSR,
    and every stored column id is the gather-layout image of the global id"""
    n, s, d = graph_case(name)
    rp, ci = O.csr_build(n, s, d, F)
    bounds = O.partition(rp, world)
    max_rows = int(np.diff(bounds).max())
    sd, dd = s.to(DEV).contiguous(), d.to(DEV).contiguous()
    rows, cols = [], []
    for r in range(world):
        g = G.granii_graph_csr_create(n, sd, dd, F, r, world)
        assert (g.info.row_begin, g.info.row_end) == (bounds[r], bounds[r + 1])
        lrp, lci = G.granii_graph_export_csr(g)
        _, lay = G.granii_graph_export_local(g)
        assert np.array_equal(lay, G.granii_gather_layout_host(lci, bounds, world, max_rows))
        rows.append(lrp[1:] + (rows[-1][-1] if rows else 0))
        cols.append(lci)
    assert np.array_equal(np.concatenate([[0]] + rows), rp)
    assert np.array_equal(np.concatenate(cols), ci)


# phases of the overlapped aggregation: "off" = all-gather then SpMM; "auto" = the cost model's P;
# "2" = own block + one chunk; "16" = one phase per block (clamped to G)
PHASES = ["off", "auto", "2", "16"]


def set_phases(monkeypatch, phases):
    monkeypatch.delenv("GRANII_COMM_PHASES", raising=False)
    monkeypatch.setenv("GRANII_COMM_OVERLAP", "0" if phases == "off" else "1")
    if phases not in ("off", "auto"):
        monkeypatch.setenv("GRANII_COMM_PHASES", phases)


@pytest.mark.parametrize("phases", PHASES)
@pytest.mark.parametrize("world", [2, 3, 4])
@pytest.mark.parametrize("comp", [0, 1, 2, 3])
@pytest.mark.parametrize("name,K1,K2", [("sparse", 32, 48), ("dense", 64, 24), ("tiny", 3, 5)])
def test_gcn_forward_backward_partitioned(G, world, comp, name, K1, K2, phases, monkeypatch):
    from paper_conf_cgo_lenadorasgytm26_b200.model import GNN, LayerSpec
    set_phases(monkeypatch, phases)
    n, s, d = graph_case(name)
    rp, ci = O.csr_build(n, s, d, F)
    H = synth.features(90, n, K1)
    W = synth.glorot(90, 2, K1, K2, (K1, K2))
    Gup = synth.uniform_pm1(90, 3, (n, K2))

    def body(r, g, comm, rows):
        b0, b1 = rows
        net = GNN(g, [LayerSpec(G.GCN, K1, K2, G.ACT_RELU, comp=comp, W=W.to(DEV))], DEV, comm=comm)
        out = net.forward(padded(H[b0:b1]))
        dH = net.backward(padded(Gup[b0:b1]), need_input_grad=True)
        return out.cpu(), dH.cpu(), net.dW[0].cpu()

    res, _ = run_ranks(G, world, n, s, d, body)
    ref, _ = O.gcn_forward(comp, rp, ci, H, W, 1)
    rdH, rdW = O.gcn_backward(comp, rp, ci, H, W, Gup, 1)
    assert err(torch.cat([x[0] for x in res]), ref) <= TOL
    assert err(torch.cat([x[1] for x in res]), rdH) <= TOL
    for r in range(world):  # dW all-reduced: every rank holds the same (bitwise) full gradient
        assert err(res[r][2], rdW) <= TOL
        assert torch.equal(res[r][2], res[0][2])


@pytest.mark.parametrize("tile", ["auto", "1"])
@pytest.mark.parametrize("phases", ["off", "16"])
@pytest.mark.parametrize("world", [2, 4])
@pytest.mark.parametrize("comp", [16, 17])
@pytest.mark.parametrize("name,K1,K2", [("sparse", 32, 64), ("dense", 48, 16)])
def test_gat_forward_backward_partitioned(G, world, comp, name, K1, K2, phases, tile, monkeypatch):
    """tile = 1 forces the entry-tile K = 1 SDDMM (chosen on its own only for products-sized graphs) over
    the partitioned graph: local rows, gather-layout column ids, cut rows at tile boundaries"""
    from paper_conf_cgo_lenadorasgytm26_b200.model import GNN, LayerSpec
    set_phases(monkeypatch, phases)
    if tile != "auto":
        monkeypatch.setenv("GRANII_SDDMM_TILE", tile)
    n, s, d = graph_case(name)
    rp, ci = O.csr_build(n, s, d, F)
    H = synth.features(91, n, K1)
    W = synth.glorot(91, 2, K1, K2, (K1, K2))
    al = synth.uniform_pm1(91, 3, (K2,))
    ar = synth.uniform_pm1(91, 4, (K2,))
    Gup = synth.uniform_pm1(91, 5, (n, K2))

    def body(r, g, comm, rows):
        b0, b1 = rows
        spec = LayerSpec(G.GAT, K1, K2, G.ACT_NONE, comp=comp, W=W.to(DEV), a_l=al.to(DEV), a_r=ar.to(DEV))
        net = GNN(g, [spec], DEV, comm=comm)
        out = net.forward(padded(H[b0:b1]))
        dH = net.backward(padded(Gup[b0:b1]), need_input_grad=True)
        return out.cpu(), dH.cpu(), net.dW[0].cpu(), net.da[0][0].cpu(), net.da[0][1].cpu()

    res, _ = run_ranks(G, world, n, s, d, body)
    ref, _ = O.gat_forward(comp, rp, ci, H, W, al, ar, 0)
    assert err(torch.cat([x[0] for x in res]), ref) <= TOL
    rg = O.gat_backward(comp, rp, ci, H, W, al, ar, Gup, 0)
    mag = O.gat_backward_magnitude(comp, rp, ci, H, W, al, ar, Gup, 0)
    assert gat_grad_ok(torch.cat([x[1] for x in res]), rg[0], mag[0]), "dH"
    for r in range(world):
        for i, nm in ((2, "dW"), (3, "da_l"), (4, "da_r")):
            assert gat_grad_ok(res[r][i], rg[i - 1], mag[i - 1]), (r, nm)
            assert torch.equal(res[r][i], res[0][i]), (r, nm)


@pytest.mark.parametrize("phases", ["2", "3", "16"])
@pytest.mark.parametrize("world", [3, 8])
def test_phased_spmm_segments_slices_deterministic(G, world, phases, monkeypatch):
    """the block-phased aggregation with hub segments (GRANII_SEG=64: partials carried across
    the phases, combined after the last) and forced K slices; bitwise reproducible"""
    from paper_conf_cgo_lenadorasgytm26_b200.model import GNN, LayerSpec
    n, s, d = graph_case("dense")
    rp, ci = O.csr_build(n, s, d, F)
    K1, K2 = 72, 40
    H = synth.features(94, n, K1)
    W = synth.glorot(94, 2, K1, K2, (K1, K2))
    Gup = synth.uniform_pm1(94, 3, (n, K2))
    monkeypatch.setenv("GRANII_SEG", "64")
    monkeypatch.setenv("GRANII_SPMM_SLICE", "16")
    set_phases(monkeypatch, phases)
    for comp in (0, 1, 2, 3):
        def body(r, g, comm, rows):
            b0, b1 = rows
            outs = []
            for _ in range(2):
                net = GNN(g, [LayerSpec(G.GCN, K1, K2, G.ACT_RELU, comp=comp, W=W.to(DEV))], DEV, comm=comm)
                out = net.forward(padded(H[b0:b1]))
                dH = net.backward(padded(Gup[b0:b1]), need_input_grad=True)
                outs.append((out.cpu(), dH.cpu()))
            return outs
        res, _ = run_ranks(G, world, n, s, d, body)
        ref, _ = O.gcn_forward(comp, rp, ci, H, W, 1)
        rdH, _ = O.gcn_backward(comp, rp, ci, H, W, Gup, 1)
        assert err(torch.cat([x[0][0] for x in res]), ref) <= TOL, comp
        assert err(torch.cat([x[0][1] for x in res]), rdH) <= TOL, comp
        for x in res:
            assert torch.equal(x[0][0], x[1][0]) and torch.equal(x[0][1], x[1][1])


@pytest.mark.parametrize("world", [2, 3])
@pytest.mark.parametrize("model,comp", [("sgc", 32), ("sgc", 35), ("tagcn", 49), ("tagcn", 50), ("gin", 64),
                                        ("gin", 67)])
def test_ext_models_partitioned(G, world, model, comp):
    """N3 forwards: multi-hop chains all-gather between hops"""
    from paper_conf_cgo_lenadorasgytm26_b200.model import GNN, LayerSpec
    n, s, d = graph_case("sparse")
    rp, ci = O.csr_build(n, s, d, F)
    K1, K2, hops, Kh = 24, 16, 3, 20
    H = synth.features(92, n, K1)
    if model == "sgc":
        W = synth.glorot(92, 2, K1, K2, (K1, K2))
        spec = lambda: LayerSpec(G.SGC, K1, K2, 1, comp=comp, W=W.to(DEV), hops=hops)  # noqa: E731
        ref = O.sgc_forward(comp, rp, ci, H, W, hops, 1)
        pre = O.sgc_forward(comp, rp, ci, H, W, hops, 0)
    elif model == "tagcn":
        Ws = synth.glorot(92, 2, K1, K2, (hops + 1, K1, K2))
        spec = lambda: LayerSpec(G.TAGCN, K1, K2, 1, comp=comp, W=Ws.to(DEV).contiguous(), hops=hops)  # noqa: E731
        ref = O.tagcn_forward(comp, rp, ci, H, Ws, 1)
        pre = O.tagcn_forward(comp, rp, ci, H, Ws, 0)
    else:
        W1 = synth.glorot(92, 2, K1, Kh, (K1, Kh))
        W2 = synth.glorot(92, 3, Kh, K2, (Kh, K2))
        spec = lambda: LayerSpec(G.GIN, K1, K2, 1, comp=comp, W=W1.to(DEV), eps=0.25, Kh=Kh,  # noqa: E731
                                 W2=W2.to(DEV))
        ref = O.gin_forward(comp, rp, ci, H, W1, W2, 0.25, 1)
        pre = O.gin_forward(comp, rp, ci, H, W1, W2, 0.25, 0)

    def body(r, g, comm, rows):
        b0, b1 = rows
        net = GNN(g, [spec()], DEV, comm=comm)
        return net.forward(padded(H[b0:b1])).cpu()

    res, _ = run_ranks(G, world, n, s, d, body)
    assert err_act(torch.cat(res), ref, pre) <= TOL


def test_comm_aware_selection(G, monkeypatch):
    """N1: on a partitioned graph the cost of every aggregation includes the all-gather of its
    operand (N x K x 4 B x (G-1)/G received per GPU), overlapped with the block-phased SpMM"""
    n, s, d = graph_case("sparse")
    world = 8
    g = G.granii_graph_csr_create(n, s.to(DEV).contiguous(), d.to(DEV).contiguous(), F, 3, world)
    name, f = G.granii_cost_features(g, 9, 64)   # P_ALLGATHER at K = 64
    assert name == "allgather"
    ncols = world * g.info.max_local_rows
    assert f[1] == pytest.approx(ncols * 64 * 4 * (world - 1) / world * 1e-9, rel=1e-12)
    for model, K1, K2 in ((G.GAT, 32, 512), (G.GCN, 256, 64), (G.GCN, 64, 256)):
        _, p_on = G.granii_select(g, model, K1, K2)
        monkeypatch.setenv("GRANII_COMM_OVERLAP", "0")
        _, p_off = G.granii_select(g, model, K1, K2)
        monkeypatch.delenv("GRANII_COMM_OVERLAP")
        assert set(p_on) == set(p_off)
        for k in p_on:  # hiding the transfer can only lower the predicted time
            assert p_off[k] >= p_on[k] - 1e-12, (model, k)


@pytest.mark.parametrize("name", ["sparse", "dense"])
def test_selection_identical_on_every_rank(G, name, monkeypatch):
    """the compositions issue different collectives, so every rank of a partition must select the
    same one: the selector's inputs on a partitioned graph are whole-graph quantities"""
    n, s, d = graph_case(name)
    monkeypatch.setenv("GRANII_SEG", "64")   # hub segments exist and are unevenly spread over ranks
    sd, dd = s.to(DEV).contiguous(), d.to(DEV).contiguous()
    for world in (2, 5, 8):
        gs = [G.granii_graph_csr_create(n, sd, dd, F, r, world) for r in range(world)]
        for model, K1, K2, fl in ((G.GCN, 64, 256, 0), (G.GCN, 256, 64, G.SELECT_TRAINING),
                                  (G.GAT, 32, 128, G.SELECT_TRAINING | G.SELECT_INPUT_LAYER)):
            picks = [G.granii_select(g, model, K1, K2, flags=fl) for g in gs]
            assert all(p == picks[0] for p in picks), (world, model, picks)


def test_comm_stats_count_the_exchanged_bytes(G):
    """granii_comm_stats: a DYN_UPD forward on a G-way partition receives (G-1) blocks of the
    K2-wide gather buffer per rank (block broadcasts), the backward the same again plus the
    ring all-reduce of dW"""
    from paper_conf_cgo_lenadorasgytm26_b200.model import GNN, LayerSpec
    n, s, d = graph_case("sparse")
    world, K1, K2 = 4, 16, 24
    W = synth.glorot(95, 2, K1, K2, (K1, K2))

    os.environ["GRANII_COMM_PHASES"] = "16"   # one broadcast per block in every regime

    def body(r, g, comm, rows):
        b0, b1 = rows
        net = GNN(g, [LayerSpec(G.GCN, K1, K2, G.ACT_RELU, comp=3, W=W.to(DEV))], DEV, comm=comm)
        net.forward(padded(synth.features(95, n, K1)[b0:b1]))
        f = G.granii_comm_stats(comm)
        net.backward(padded(synth.uniform_pm1(95, 3, (n, K2))[b0:b1]), need_input_grad=False)
        return f, G.granii_comm_stats(comm), g.info.max_local_rows

    try:
        res, _ = run_ranks(G, world, n, s, d, body)
    finally:
        os.environ.pop("GRANII_COMM_PHASES", None)
    for (fb, fc), (bb, bc), mr in res:
        ld = (K2 + 7) // 8 * 8
        assert fb == (world - 1) * mr * ld * 4 and fc == world
        assert bb - fb == (world - 1) * mr * ld * 4 + int(2.0 * K1 * K2 * 4 * (world - 1) / world)


def test_comm_collectives_nccl_one_rank_and_loopback(G):
    """The public collectives through both real transports: a 1-rank NCCL communicator (the library
    dlopens the NCCL PyTorch loaded and calls ncclAllGather / ncclAllReduce on the caller's stream;
    one rank is all a single-GPU box can form) and a 3-rank loopback group (one thread per rank)"""
    n = 1000
    x = torch.arange(n, dtype=torch.float32, device=DEV)
    comm = G.granii_comm_create(G.granii_comm_unique_id(), 0, 1)
    recv = torch.full((n,), -1.0, device=DEV)
    G.granii_comm_allgather(comm, x, recv, n)
    buf = x.clone()
    G.granii_comm_allgather(comm, buf, buf, n)  # in place
    red = x.clone()
    G.granii_comm_allreduce_sum(comm, red)
    torch.cuda.synchronize()
    assert torch.equal(recv, x) and torch.equal(buf, x) and torch.equal(red, x)
    del comm
    world = 3
    comms = G.granii_comm_create_local(world)
    outs, sums, errs = [None] * world, [None] * world, []

    def worker(r):
        try:
            torch.cuda.set_device(DEV)
            st = torch.cuda.Stream(device=DEV)
            with torch.cuda.stream(st):
                all_ = torch.zeros(world * n, device=DEV)
                all_[r * n:(r + 1) * n] = x + 1000.0 * r
                G.granii_comm_allgather(comms[r], all_[r * n:(r + 1) * n], all_, n, st)
                v = x * (r + 1)
                G.granii_comm_allreduce_sum(comms[r], v, st)
            st.synchronize()
            outs[r], sums[r] = all_.cpu(), v.cpu()
        except Exception as e:  # pragma: no cover - surfaced below
            errs.append(e)
    th = [threading.Thread(target=worker, args=(r,)) for r in range(world)]
    for t in th:
        t.start()
    for t in th:
        t.join()
    assert not errs, errs
    want = torch.cat([x.cpu() + 1000.0 * r for r in range(world)])
    for r in range(world):
        assert torch.equal(outs[r], want)
        assert torch.equal(sums[r], x.cpu() * 6)


def test_comm_query_register_and_watchdog_no_false_alarm(G):
    """A 1-rank NCCL communicator reports nranks = 1 / rank 0 through ncclCommCount /
    ncclCommUserRank; a registered buffer works as a collective operand; with the watchdog
    running, collectives that complete never trip it"""
    comm = G.granii_comm_create(G.granii_comm_unique_id(), 0, 1)
    n, r, v = G.granii_comm_query(comm)
    assert (n, r) == (1, 0) and v >= 21800          # NCCL 2.18+ encodes 2.18.0 as 21800
    buf = torch.arange(4096, dtype=torch.float32, device=DEV)
    try:
        h = G.granii_comm_register(comm, buf)
    except G.GraniiError as e:                      # NCCL without user-buffer registration
        assert "ncclCommRegister" in str(e)
        h = None
    G.granii_comm_watchdog(comm, 2000)
    want = buf.clone()
    for _ in range(50):
        G.granii_comm_allreduce_sum(comm, buf)
    torch.cuda.synchronize()
    time.sleep(0.1)
    G.granii_comm_check(comm)
    assert torch.equal(buf, want)
    if h is not None:
        G.granii_comm_deregister(comm, h)
    G.granii_comm_watchdog(comm, 0)
    del comm


def test_comm_watchdog_aborts_a_stuck_collective(G):
    """Failure detection: a collective held back on the device longer than the watchdog timeout
    (here by a 1.5 s kernel queued before it on the same stream, standing in for a peer that
    never arrives) aborts the communicator, and later calls fail with the reason instead of
    hanging.  Loopback transport, so the abort is a flag and the GPU stays healthy."""
    comm = G.granii_comm_create_local(1)[0]
    G.granii_comm_watchdog(comm, 200)
    x = torch.ones(1024, device=DEV)
    G.granii_comm_allreduce_sum(comm, x)      # first call sizes the staging buffer (a host sync)
    torch.cuda.synchronize()
    time.sleep(0.3)
    G.granii_comm_check(comm)                 # completed collectives never trip it
    G.granii_debug_spin(1_500_000)
    G.granii_comm_allreduce_sum(comm, x)
    time.sleep(0.8)
    with pytest.raises(G.GraniiError, match="pending"):
        G.granii_comm_check(comm)
    with pytest.raises(G.GraniiError, match="watchdog"):
        G.granii_comm_allreduce_sum(comm, x)
    torch.cuda.synchronize()
    G.granii_comm_watchdog(comm, 0)


@pytest.mark.parametrize("world", [2, 3])
@pytest.mark.parametrize("comp", [0, 1, 2, 3, 16, 17])
def test_directed_backward_partitioned(G, world, comp, monkeypatch):
    """GRANII_BUILD_TRANSPOSE on a partitioned directed (R-MAT) graph: every rank keeps its rows of
    Ãᵀ over Ã's row block, in the same gather layout; the transposed aggregations of the GCN and
    GAT backward run over them (forced one-phase-per-block to exercise the phased Ãᵀ SpMM)"""
    from paper_conf_cgo_lenadorasgytm26_b200.model import GNN, LayerSpec
    set_phases(monkeypatch, "16")
    n = 1200
    s, d = synth.rmat(n, 9000, 0.57, 0.19, 0.19, seed=26)
    fl = G.ADD_SELF_LOOPS | G.BUILD_TRANSPOSE
    rp, ci = O.csr_build(n, s, d, O.ADD_SELF_LOOPS)
    rpt, cit = O.csr_build(n, d, s, O.ADD_SELF_LOOPS)       # Ãᵀ: the reversed edges
    bounds = O.partition(rp, world)
    K1, K2 = 24, 40
    H = synth.features(97, n, K1)
    W = synth.glorot(97, 2, K1, K2, (K1, K2))
    al = synth.uniform_pm1(97, 3, (K2,))
    ar = synth.uniform_pm1(97, 4, (K2,))
    Gup = synth.uniform_pm1(97, 5, (n, K2))
    gat = comp >= 16
    if not gat:
        _, Y = O.gcn_forward(comp, rp, ci, H, W, 1)
        Gup[torch.from_numpy(np.abs(Y) < 1e-4 * np.abs(Y).max())] = 0.0   # R20

    def body(r, g, comm, rows):
        b0, b1 = rows
        trp, tci = G.granii_graph_export_transpose(g)
        if gat:
            spec = LayerSpec(G.GAT, K1, K2, G.ACT_NONE, comp=comp, W=W.to(DEV), a_l=al.to(DEV), a_r=ar.to(DEV))
        else:
            spec = LayerSpec(G.GCN, K1, K2, G.ACT_RELU, comp=comp, W=W.to(DEV))
        net = GNN(g, [spec], DEV, comm=comm)
        net.forward(padded(H[b0:b1]))
        dH = net.backward(padded(Gup[b0:b1]), need_input_grad=True)
        da = (net.da[0][0].cpu(), net.da[0][1].cpu()) if gat else (None, None)
        return (trp, tci), dH.cpu(), net.dW[0].cpu(), da[0], da[1]

    res, _ = run_ranks(G, world, n, s, d, body, flags=fl)
    for r in range(world):                                  # Ãᵀ rows of the block, bit-exact
        b0, b1 = int(bounds[r]), int(bounds[r + 1])
        trp, tci = res[r][0]
        assert np.array_equal(trp, rpt[b0:b1 + 1] - rpt[b0]) and np.array_equal(tci, cit[rpt[b0]:rpt[b1]])
    dH = torch.cat([x[1] for x in res])
    if gat:
        rg = O.gat_backward(comp, rp, ci, H, W, al, ar, Gup, 0)
        mag = O.gat_backward_magnitude(comp, rp, ci, H, W, al, ar, Gup, 0)
        assert gat_grad_ok(dH, rg[0], mag[0]), "dH"
        for r in range(world):
            for i, nm in ((2, "dW"), (3, "da_l"), (4, "da_r")):
                assert gat_grad_ok(res[r][i], rg[i - 1], mag[i - 1]), (r, nm)
    else:
        rdH, rdW = O.gcn_backward(comp, rp, ci, H, W, Gup, 1)
        assert err(dH, rdH) <= TOL
        for r in range(world):
            assert err(res[r][2], rdW) <= TOL
