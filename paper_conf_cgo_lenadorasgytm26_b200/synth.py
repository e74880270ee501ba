"""Seeded synthetic inputs shared by the oracle tests and the CUDA path.

This module is the ONLY code both sides of a parity check share.  It holds none
of the method's arithmetic: no normalisation, no aggregation, no attention, no
CSR construction.  It only draws integers and floats from a counter-based
generator and shapes them like the paper's workloads.

Everything is integer hashing (splitmix64 on int64 tensors, wrap-around
multiply) so a generator run on CPU and on CUDA gives bit-identical output.
Floats are built from <= 24 random bits, so they are exact in fp32.

Workload shapes follow PAPER.md Table II (L292-L301: Reddit 232,965 nodes /
114,615,892 edges, ogbn-products 2,449,029 / 126,167,053, ...) and
BASELINE.json `configs` (Cora-, Pubmed-, ogbn-arxiv-, Reddit-, ogbn-products-
shaped graphs).  The paper's graphs are undirected and unweighted (L328), so
undirected workloads are emitted as one directed (src, dst) per pair and the
CSR builder's SYMMETRIZE flag adds the reverse entry.  Recipe: DESIGN.md §3.
"""
from __future__ import annotations

import math
from dataclasses import dataclass, field

import torch

_GOLDEN = -7046029254386353131          # 0x9E3779B97F4A7C15 as int64
_M1 = -4658895280553007687              # 0xBF58476D1CE4E5B9
_M2 = -7723592293110705685              # 0x94D049BB133111EB


def _srl(x: torch.Tensor, s: int) -> torch.Tensor:
    """Logical right shift of an int64 tensor."""
    return (x >> s) & ((1 << (64 - s)) - 1)


def splitmix64(x: torch.Tensor) -> torch.Tensor:
    """splitmix64 finaliser on int64 (two's-complement wrap-around)."""
    z = x + _GOLDEN
    z = (z ^ _srl(z, 30)) * _M1
    z = (z ^ _srl(z, 27)) * _M2
    return z ^ _srl(z, 31)


def stream_bits(seed: int, stream: int, n: int, device="cpu", offset: int = 0) -> torch.Tensor:
    """n pseudo-random int64 words; word i = splitmix64(key + i)."""
    key = splitmix64(torch.tensor([seed * 1_000_003 + stream * 7_919 + 12345], dtype=torch.int64))
    ctr = torch.arange(offset, offset + n, dtype=torch.int64, device=device)
    return splitmix64(ctr + int(key.item()))


def uniform_int(seed: int, stream: int, n: int, bound: int, device="cpu") -> torch.Tensor:
    """n integers uniform in [0, bound) (bound < 2^40), from the top 40 bits."""
    r = _srl(stream_bits(seed, stream, n, device), 24)
    return r % bound


def uniform_pm1(seed: int, stream: int, shape, device="cpu") -> torch.Tensor:
    """fp32 tensor uniform in [-1, 1): (u24 / 2^23) - 1, exact in fp32."""
    n = int(math.prod(shape))
    u = _srl(stream_bits(seed, stream, n, device), 40)          # 24 bits
    return (u.to(torch.float32) * (1.0 / 8388608.0) - 1.0).reshape(shape)


def glorot(seed: int, stream: int, fan_in: int, fan_out: int, shape, device="cpu") -> torch.Tensor:
    """Glorot-uniform weights +-sqrt(6/(fan_in+fan_out)) (reading R15)."""
    lim = torch.tensor(math.sqrt(6.0 / (fan_in + fan_out)), dtype=torch.float32)
    return uniform_pm1(seed, stream, shape, device) * lim.to(device)


# ---------------------------------------------------------------- graphs

def chung_lu(n: int, m: int, gamma: float, seed: int, device="cpu", max_w_frac: float = 0.05):
    """m directed (src, dst) draws of a Chung-Lu graph on n nodes.

    Node weights follow a power law w_i ~ (i + i0)^(-1/(gamma-1)); they are
    rounded to integers on the host so the cumulative table is exact on any
    device.  Each endpoint is drawn by inverse CDF over that table, then node
    ids are relabelled by a seeded permutation (no id locality).
    """
    i = torch.arange(n, dtype=torch.float64)
    i0 = max(1.0, n * 1e-4)
    w = (i + i0) ** (-1.0 / (gamma - 1.0))
    w = w / w.sum()
    w = torch.clamp(w, max=max_w_frac)                  # caps the largest hub
    wi = torch.clamp((w * (2 ** 40)).round().to(torch.int64), min=1)
    cdf = torch.cumsum(wi, 0).to(device)
    total = int(cdf[-1].item())
    perm = _permutation(n, seed, 9, device)
    u = uniform_int(seed, 1, m, total, device)
    v = uniform_int(seed, 2, m, total, device)
    src = torch.searchsorted(cdf, u, right=True)
    dst = torch.searchsorted(cdf, v, right=True)
    return perm[src].to(torch.int32), perm[dst].to(torch.int32)


def rmat(n: int, m: int, a: float, b: float, c: float, seed: int, device="cpu"):
    """m directed R-MAT draws (Chakrabarti et al.) mapped onto [0, n).

    Quadrant probabilities (a, b, c, 1-a-b-c) are quantised to 1/65536.  Ids
    of the 2^scale grid are scaled into [0, n) and relabelled by a seeded
    permutation.
    """
    scale = max(1, math.ceil(math.log2(n)))
    ta, tb, tc = int(a * 65536), int((a + b) * 65536), int((a + b + c) * 65536)
    src = torch.zeros(m, dtype=torch.int64, device=device)
    dst = torch.zeros(m, dtype=torch.int64, device=device)
    for lvl in range(scale):
        r = _srl(stream_bits(seed, 100 + lvl, m, device), 48)      # 16 bits
        right = ((r >= ta) & (r < tb)) | (r >= tc)                  # quadrants b, d
        down = r >= tb                                              # quadrants c, d
        src = (src << 1) | down.to(torch.int64)
        dst = (dst << 1) | right.to(torch.int64)
    src = (src * n) >> scale
    dst = (dst * n) >> scale
    perm = _permutation(n, seed, 99, device)
    return perm[src].to(torch.int32), perm[dst].to(torch.int32)


def _permutation(n: int, seed: int, stream: int, device) -> torch.Tensor:
    keys = stream_bits(seed, stream, n, device)
    # ties are broken by index (stable) so the permutation is device-independent
    return torch.sort(keys, stable=True).indices


def road(n: int, seed: int, device="cpu", p_extra: float = 0.05):
    """Road-network-like graph (belgium_osm shape, Table II): a near-square
    grid lattice (right / down neighbours, ids in grid order: spatial locality)
    with a seeded fraction of lattice edges dropped and a few random shortcuts,
    giving average degree ~3 and a near-uniform degree distribution."""
    side = int(math.ceil(math.sqrt(n)))
    i = torch.arange(n, dtype=torch.int64, device=device)
    r, c = i // side, i % side
    right = (c + 1 < side) & (i + 1 < n)
    down = i + side < n
    src = torch.cat([i[right], i[down]])
    dst = torch.cat([i[right] + 1, i[down] + side])
    keep = uniform_int(seed, 30, src.numel(), 1000, device) >= 300          # drop 30% of lattice edges
    src, dst = src[keep], dst[keep]
    k = int(p_extra * n)
    es = uniform_int(seed, 31, k, n, device)
    ed = torch.clamp(es + uniform_int(seed, 32, k, 64, device) - 32, 0, n - 1)  # short random links
    return torch.cat([src, es]).to(torch.int32), torch.cat([dst, ed]).to(torch.int32)


def ring(n: int, k: int):
    """k-regular ring lattice (k even): i -> i+1..i+k/2, undirected pairs."""
    src = torch.arange(n, dtype=torch.int64).repeat_interleave(k // 2)
    off = torch.arange(1, k // 2 + 1, dtype=torch.int64).repeat(n)
    return src.to(torch.int32), ((src + off) % n).to(torch.int32)


def complete(n: int):
    """Complete graph K_n as undirected pairs (i < j)."""
    ii, jj = torch.triu_indices(n, n, offset=1)
    return ii.to(torch.int32), jj.to(torch.int32)


def random_small(n: int, m: int, seed: int):
    """Uniform random directed edges (for tiny adversarial tests)."""
    return (uniform_int(seed, 5, m, n).to(torch.int32),
            uniform_int(seed, 6, m, n).to(torch.int32))


# ---------------------------------------------------------------- workloads

@dataclass
class Workload:
    name: str
    n: int
    m: int                      # directed draws fed to the builder
    kind: str                   # "chung_lu" | "rmat"
    symmetrize: bool
    gamma: float = 2.5
    rmat_abc: tuple = (0.57, 0.19, 0.19)
    max_w_frac: float = 0.05
    dims: dict = field(default_factory=dict)
    cite: str = ""

    def edges(self, seed: int = 0, device="cpu"):
        if self.kind == "chung_lu":
            return chung_lu(self.n, self.m, self.gamma, seed, device, self.max_w_frac)
        if self.kind == "road":
            return road(self.n, seed, device)
        a, b, c = self.rmat_abc
        return rmat(self.n, self.m, a, b, c, seed, device)


# Shapes: BASELINE.json configs + PAPER.md Table II (L292-L301), Table IV dims (L375-L386).
WORKLOADS = {
    # configs[0]: Cora-shaped, 2,708 nodes, ~10.5k directed edges, 1433 -> 16
    "cora": Workload("cora", 2708, 5278, "chung_lu", True, gamma=2.5,
                     dims={"K1": 1433, "K2": 16}, cite="BASELINE.json configs[0]"),
    # configs[1]: Pubmed-shaped, 19.7k nodes, ~88k directed edges, emb 32/256
    "pubmed": Workload("pubmed", 19717, 44324, "chung_lu", True, gamma=2.5,
                       dims={"K": [32, 256]}, cite="BASELINE.json configs[1]"),
    # configs[2]: ogbn-arxiv-shaped power-law graph, 169k nodes, 1.17M directed edges
    "arxiv": Workload("arxiv", 169343, 1166243, "rmat", False,
                      dims={"pairs": [(64, 128), (64, 256), (64, 512), (128, 256), (128, 512), (256, 512)]},
                      cite="BASELINE.json configs[2]"),
    # configs[3]: Reddit-shaped dense-degree graph, 232,965 nodes, 114,615,892 directed edges
    "reddit": Workload("reddit", 232965, 59_500_000, "chung_lu", True, gamma=2.9, max_w_frac=0.0004,
                       dims={"K_in": 602, "K_hid": [32, 256, 1024], "K_out": 41},
                       cite="PAPER.md Table II L296, Table IV L375-L377"),
    # configs[4]: ogbn-products-shaped, 2,449,029 nodes, 126,167,053 directed edges
    "products": Workload("products", 2449029, 64_000_000, "rmat", True, rmat_abc=(0.45, 0.22, 0.22),
                         dims={"K_in": 100, "K_hid": [32, 256, 1024], "K_out": 47},
                         cite="PAPER.md Table II L301, Table IV L381-L386"),
    # selector-regret extremes of Table II: road-like and very dense
    "belgium": Workload("belgium", 1441295, 0, "road", True, dims={"K": [32, 256, 1024]},
                        cite="PAPER.md Table II L299 (belgium_osm: 1,441,295 nodes, 4,541,235 edges)"),
    "mycielskian": Workload("mycielskian", 98303, 52_000_000, "chung_lu", True, gamma=4.0, max_w_frac=0.0005,
                            dims={"K": [32, 256, 1024]},
                            cite="PAPER.md Table II L298 (mycielskian17: 98,303 nodes, 100,245,742 edges)"),
}


def features(seed: int, n: int, k: int, device="cpu", ld: int | None = None) -> torch.Tensor:
    """Node features H ~ U(-1, 1), fp32, shape (n, k); optional padded row stride ld."""
    ld = ld or k
    x = uniform_pm1(seed, 11, (n, ld), device)
    if ld != k:
        x[:, k:] = 0.0
    return x if ld == k else x[:, :k]


def labels(seed: int, n: int, classes: int, device="cpu") -> torch.Tensor:
    return uniform_int(seed, 13, n, classes, device).to(torch.int32)
