"""Multi-layer GNN driver over the C ABI (§VI-F, Fig. 4).

GRANII selects one composition per layer from the input graph and the layer's
embedding sizes, once per (graph, K1, K2), and reuses the decision across
iterations (L409).  This module only sequences ABI calls and owns the device
buffers (workspaces, activations, gradients) as torch tensors; every FLOP runs
in libgranii.so.
"""
from __future__ import annotations

import os
from dataclasses import dataclass, field

import torch

from . import granii as G

# B200 calibration of the per-primitive cost models (tools/calibrate.py)
DEFAULT_CALIB = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "calib", "b200.txt")


def _pad4(k: int) -> int:
    """row stride: 16-byte rows, whole 32-byte sectors once a row has >= 8 floats"""
    return (k + 7) // 8 * 8 if k >= 8 else (k + 3) // 4 * 4


def alloc2d(rows: int, cols: int, device, fill=None) -> torch.Tensor:
    """(rows, cols) fp32 view of a buffer whose row stride is padded to 16 bytes."""
    buf = torch.empty((max(rows, 1), _pad4(cols)), dtype=torch.float32, device=device)
    buf[:, cols:].zero_()        # padding columns: read (never used) by the float4 gathers of a ragged last vector
    if fill is not None:
        buf.fill_(fill)
    return buf[:rows, :cols]


@dataclass
class LayerSpec:
    model: int                  # G.GCN | G.GAT
    K1: int
    K2: int
    act: int = G.ACT_RELU
    attn: int = G.ATTN_ADDITIVE
    comp: int | None = None     # None -> chosen by granii_select
    W: torch.Tensor | None = None  # TAGCN: (hops+1, K1, K2) stacked; GIN: K1 x Kh
    a_l: torch.Tensor | None = None
    a_r: torch.Tensor | None = None
    hops: int = 2               # SGC / TAGCN
    eps: float = 0.0            # GIN
    Kh: int = 0                 # GIN hidden width
    W2: torch.Tensor | None = None  # GIN: Kh x K2
    predicted_ms: dict = field(default_factory=dict)


class GNN:
    """A stack of GCN/GAT layers on one (possibly row-partitioned) graph."""

    def __init__(self, graph: G.Graph, layers: list[LayerSpec], device, comm: G.Comm | None = None,
                 calib_path: str | None = None, select_flags: int = G.SELECT_REFINE, training: bool = False):
        """training=True costs each candidate's backward too (extension; the paper selects on the
        forward only, L340) and knows the input layer needs no dH.  select_flags defaults to the
        measured tie-break of near-equal predictions on small layers (GRANII_SELECT_REFINE, single
        GPU; pass 0 for the cost model alone)."""
        self.g, self.layers, self.device, self.comm = graph, layers, device, comm
        if calib_path is None and os.path.exists(DEFAULT_CALIB):
            calib_path = DEFAULT_CALIB
        for i, L in enumerate(layers):
            if L.comp is None:
                fl = select_flags
                if training:
                    fl |= G.SELECT_TRAINING | (G.SELECT_INPUT_LAYER if i == 0 else 0)
                L.comp, L.predicted_ms = G.granii_select_ex(graph, L.model, G.shape_args(L.K1, L.K2, L.hops, L.Kh),
                                                            calib_path, fl)
        ws = 0
        self.saved_floats = []
        for L in layers:
            w, s = G.granii_layer_workspace_size_ex(graph, L.model, L.comp, G.shape_args(L.K1, L.K2, L.hops, L.Kh))
            ws = max(ws, w)
            self.saved_floats.append(s)
        self.workspace = torch.empty(max(ws, 1), dtype=torch.uint8, device=device)
        # the gather buffers of the all-gathers live in the workspace: register it with NCCL so
        # collectives can use it in place (ncclCommRegister; a no-op on loopback / stub transports)
        self.nccl_handle, self.nccl_register = None, None
        if comm is not None and comm.world > 1 and os.environ.get("GRANII_NCCL_REGISTER", "1") != "0":
            try:
                self.nccl_handle = G.granii_comm_register(comm, self.workspace)
                self.nccl_register = "registered" if self.nccl_handle else "not applicable (transport)"
            except G.GraniiError as e:   # NCCL without registration support: collectives still work
                self.nccl_register = f"not registered: {e}"
        R = graph.n_rows
        self.outs = [alloc2d(R, L.K2, device) for L in layers]
        self.saved = [torch.empty(max(s, 1), dtype=torch.float32, device=device) if s else None
                      for s in self.saved_floats]
        self.grads_out = [alloc2d(R, L.K2, device) for L in layers]     # dL/d out_l
        self.dW = [torch.empty((L.K1, L.K2), dtype=torch.float32, device=device) for L in layers]
        # dL/da_l, dL/da_r of the GAT layers (None for GCN)
        self.da = [(torch.empty(L.K2, dtype=torch.float32, device=device),
                    torch.empty(L.K2, dtype=torch.float32, device=device)) if L.model == G.GAT else None
                   for L in layers]

    def __del__(self):
        if getattr(self, "nccl_handle", None) and self.comm is not None and self.comm.handle:
            try:
                G.granii_comm_deregister(self.comm, self.nccl_handle)
            except Exception:  # noqa: BLE001 -- interpreter shutdown
                pass

    def args(self, i: int, H: torch.Tensor) -> G.layer_args:
        L = self.layers[i]
        da = self.da[i] or (None, None)
        return G.make_layer_args(L.K1, L.K2, H, L.W, L.a_l, L.a_r, L.act, L.attn, self.workspace, self.comm,
                                 da[0], da[1], L.hops, L.eps, L.Kh, L.W2)

    def forward(self, H: torch.Tensor) -> torch.Tensor:
        x = H
        self._inputs = []
        for i, L in enumerate(self.layers):
            self._inputs.append(x)
            G.granii_layer_forward(self.g, L.model, L.comp, self.args(i, x), self.outs[i], self.saved[i])
            x = self.outs[i]
        return x

    def backward(self, dout_last: torch.Tensor, need_input_grad: bool = False):
        """Backward through all layers (L340; GAT additive attention, R22); fills self.dW and self.da."""
        dout = dout_last
        for i in range(len(self.layers) - 1, -1, -1):
            L = self.layers[i]
            dH = self.grads_out[i - 1] if i > 0 else (alloc2d(self.g.n_rows, L.K1, self.device)
                                                      if need_input_grad else None)
            G.granii_layer_backward(self.g, L.model, L.comp, self.args(i, self._inputs[i]), self.outs[i], dout,
                                    self.saved[i], dH, self.dW[i])
            dout = dH
        return dout

    def train_step(self, H: torch.Tensor, labels: torch.Tensor, n_total: int, lr: float,
                   dlogits: torch.Tensor, loss: torch.Tensor | None = None):
        """forward -> softmax cross-entropy -> backward -> SGD update of every W."""
        Z = self.forward(H)
        G.granii_softmax_xent(Z, labels, n_total, dlogits, loss)
        self.backward(dlogits)
        for L, dW, da in zip(self.layers, self.dW, self.da):
            G.granii_sgd(dW, L.W, lr)
            if da is not None:
                G.granii_sgd(da[0], L.a_l, lr)
                G.granii_sgd(da[1], L.a_r, lr)
        return Z
