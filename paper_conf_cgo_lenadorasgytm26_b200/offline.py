"""GRANII's offline stage (§IV-C): association-tree
generation (Algorithm 1) over a layer's matrix IR and input-oblivious pruning
(L226-L233), producing the promoted compositions the online selector chooses from.

The matrix IR of a layer is a product chain of leaves (L194, Fig. 6(c): row-broadcasts
rewritten as multiplications by diagonal matrices).  Leaf kinds: 'D' diagonal (D̃^-1/2),
'A' sparse pattern (Ã), 'S' sparse with values (α), 'X' dense (H), 'W' dense weight.

Rules for association candidates (Appendix D is not in the text; reading R24):
  * adjacent leaves only (Algorithm 1 line 2: candidates involve only leaf nodes);
  * sparse x dense -> SpMM; dense x weight -> GEMM; diagonal x dense -> row-broadcast;
  * diagonal x sparse / sparse x diagonal (including an already scaled sparse) -> a
    sparse-value scaling (SDDMM with a K = 1 operand, L41 / L119-L123);
  * D A D as a whole (Fig. 6(d) tree 1) -> SDDMM(dinv, dinv): every association of the three
    leaves yields the same sparse matrix Ñ, so those trees are one tree (de-duplication).
Each internal node records its primitive and the width of the dense operand it moves
(K1 = input, K2 = output embedding size; sparse-value primitives are O(nnz)).

Pruning (L226-L233), for each scenario '>=' (K1 >= K2) and '<' (K1 < K2) separately:
  rule 1: a tree that performs every primitive of another tree -- each at a dense width never
          smaller than the other's in this scenario -- and more primitives besides is unprofitable
          (L229's example: "SpMM and a GEMM" vs "only SpMM on the same matrix sizes"); an identical
          primitive multiset is a duplicate (the first tree is kept);
  rule 2: a tree with the same primitives as another tree but a larger dense width in at
          least one of them (and no smaller one) is unprofitable.
Trees unprofitable in BOTH scenarios are pruned; the others are promoted and annotated with
the scenarios in which they survived (the embedding-size condition of L237-L239).

For GCN this yields 12 generated / 8 pruned / 4 promoted trees -- the paper's count for GCN
(L326: "12 and 8") -- and the 4 promoted trees are exactly the library's GCN compositions
with the annotations of granii_select's prefilter (update-first iff K1 >= K2).  GAT (α fixed
by the attention over Θ = H W, chain α H W) gives 2 generated / 0 pruned (L326: "2 and 0"), both
promoted: REUSE in both scenarios, RECOMP (extra GEMM, L135; SpMM at K1) only for K1 < K2, where its
narrower SpMM can pay for the GEMM -- the sizes the paper evaluates GAT at (L330) and WiseGraph's
recompute-for-growing-sizes rule (L357).  GIN (reading R23: (Ã + εI) H W1 before the MLP's ReLU,
a sum in the IR, with the distributive rewrite (P + Q) R -> P R + Q R as an extra candidate) gives 7
generated / 3 pruned / 4 promoted: the paper counts "8 and 4" (L326); the 4 promoted trees are the
library's four GIN compositions (PRE = the sum folded into the sparse values, DYN = unweighted SpMM +
the εH term, each aggregate- or update-first) with the update-first-iff-K1 >= Kh annotation.

Host-only Python: this stage runs once per model at build time, never on the data path.
"""
from __future__ import annotations

from collections import Counter
from dataclasses import dataclass

# library composition ids (include/granii.h granii_composition)
GCN_PRE_AGG, GCN_PRE_UPD, GCN_DYN_AGG, GCN_DYN_UPD = 0, 1, 2, 3
GAT_REUSE, GAT_RECOMP = 16, 17


@dataclass(frozen=True)
class Node:
    kind: str                 # 'D' 'A' 'S' 'X' 'W'
    prim: str | None = None   # primitive producing it (None for leaves)
    kids: tuple = ()
    width: str | None = None  # dense width 'K1' / 'K2'
    name: str = ""

    def show(self) -> str:
        if not self.kids:
            return self.name
        if self.prim == "SDDMM" and self.kids == ():
            return "SDDMM(DAD)"
        if self.prim in ("SpAdd", "Add"):
            return "(" + " + ".join(k.show() for k in self.kids) + ")"
        return "(" + " ".join(k.show() for k in self.kids) + ")"


def _leaf(name: str, kind: str, width: str | None = None) -> Node:
    return Node(kind, None, (), width, name)


def _leaves(n: Node) -> list[str]:
    return [n.name] if not n.kids else [x for k in n.kids for x in _leaves(k)]


def _canon(n: Node) -> Node:
    """a sparse node made of exactly the leaves D A D is the one SDDMM(dinv, dinv) -> Ñ"""
    if not n.kids:
        return n
    kids = tuple(_canon(k) for k in n.kids)
    if n.kind == "S" and [x[0] for x in _leaves(n)] == ["D", "A", "D"]:
        return Node("S", "SDDMM", (), None, "SDDMM(DAD)")
    return Node(n.kind, n.prim, kids, n.width, n.name)


def _candidates(seq: list[Node]) -> list[tuple[int, int, Node]]:
    """rule-based association candidates over adjacent nodes (Algorithm 1 line 2)"""
    out = []
    for i in range(len(seq) - 1):
        a, b = seq[i], seq[i + 1]
        if i + 2 < len(seq) and (a.kind, b.kind, seq[i + 2].kind) == ("D", "A", "D"):
            out.append((i, 3, Node("S", "SDDMM", (a, b, seq[i + 2]))))
        if a.kind in "AS" and b.kind == "X":
            out.append((i, 2, Node("X", "SpMM", (a, b), b.width)))
        elif a.kind == "X" and b.kind == "W":
            out.append((i, 2, Node("X", "GEMM", (a, b), "K2")))
        elif a.kind == "D" and b.kind == "X":
            out.append((i, 2, Node("X", "RowB", (a, b), b.width)))
        elif (a.kind == "D" and b.kind in "AS") or (a.kind in "AS" and b.kind == "D"):
            out.append((i, 2, Node("S", "SDDMM", (a, b))))
    return out


def generate(chain: list[Node]) -> list[Node]:
    """Algorithm 1 (L204-L219): depth-first over every candidate; the forest is de-duplicated
    (the same tree reached through different association orders, and the D A D equivalence)"""
    forest: list[Node] = []

    def rec(seq):
        cands = _candidates(seq)
        if not cands:
            forest.append(seq[0] if len(seq) == 1 else Node("?", None, tuple(seq)))
            return
        for i, k, node in cands:
            rec(seq[:i] + [node] + seq[i + k:])

    rec(list(chain))
    seen, out = set(), []
    for t in forest:
        c = _canon(t)
        key = c.show()
        if key not in seen:
            seen.add(key)
            out.append(c)
    return out


def primitives(t: Node, attention: bool = False) -> Counter:
    """multiset of (primitive, size) of a tree; sparse-value primitives are O(nnz) ('E'),
    every GEMM is N x K1 x K2 here, SpMM / row-broadcast carry their dense width.
    attention: the tree's α comes from the GAT scores over Θ = H W (Eq. 4): one
    GEMM for Θ -- shared with the tree's own H W node when it has one (the common
    sub-expression elimination of L219) -- and the score SDDMM"""
    c: Counter = Counter()
    if attention:
        c[("SDDMM", "E")] += 1
        if "(H W)" not in t.show():
            c[("GEMM", "K1K2")] += 1

    seen = set()  # common sub-expressions (L219): an identical subtree is computed once

    def rec(n: Node):
        if n.kids:
            key = n.show()
            if key in seen:
                return
            seen.add(key)
        if n.prim in ("SDDMM", "SpAdd"):
            c[(n.prim, "E")] += 1
        elif n.prim == "GEMM":
            c[("GEMM", "K1K2")] += 1
        elif n.prim in ("SpMM", "RowB", "Add"):
            c[(n.prim, n.width)] += 1
        for k in n.kids:
            rec(k)

    rec(t)
    return c


def _smaller(a: str, b: str, scen: str) -> bool:
    """dense width a strictly smaller than b in scenario '>=' (K1 >= K2) or '<' (K1 < K2)"""
    if a == b or a not in ("K1", "K2"):
        return False
    return (a == "K2") if scen == ">=" else (a == "K1")


def _size(w: str | None, scen: str) -> int:
    """order of the dense widths in a scenario (0 = the smaller one); unsized primitives are 0"""
    if w not in ("K1", "K2"):
        return 0
    return int(w == "K1") if scen == ">=" else int(w == "K2")


def _covers(ci: Counter, cj: Counter, scen: str) -> bool:
    """every primitive of cj matched by a distinct one of ci of the same kind, never smaller"""
    for kind in {k for k, _ in cj.elements()}:
        wi = sorted((_size(w, scen) for k, w in ci.elements() if k == kind), reverse=True)
        wj = sorted((_size(w, scen) for k, w in cj.elements() if k == kind), reverse=True)
        if len(wi) < len(wj) or any(x < y for x, y in zip(wi, wj)):
            return False
    return True


def unprofitable(i: int, trees: list[Node], scen: str, attention: bool = False) -> str | None:
    ci = primitives(trees[i], attention)
    for j, t in enumerate(trees):
        if j == i:
            continue
        cj = primitives(t, attention)
        # rule 1: I perform all of another tree's primitives, never on smaller matrices, and more
        # besides; an identical multiset is a duplicate (the first tree is kept)
        if (ci == cj and j < i) or (sum(ci.values()) > sum(cj.values()) and _covers(ci, cj, scen)):
            return f"rule 1 vs {t.show()}"
        # rule 2: same primitives, the other never larger and somewhere smaller
        ti, tj = sorted(ci.elements()), sorted(cj.elements())
        if [p for p, _ in ti] != [p for p, _ in tj]:
            continue
        strict, worse = False, False
        for typ in {p for p, _ in ti}:
            wi = sorted((w for p, w in ti if p == typ), key=lambda w: (w != "K2") == (scen == ">="))
            wj = sorted((w for p, w in tj if p == typ), key=lambda w: (w != "K2") == (scen == ">="))
            for x, y in zip(wi, wj):
                if _smaller(y, x, scen):
                    strict = True
                elif _smaller(x, y, scen):
                    worse = True
        if strict and not worse:
            return f"rule 2 vs {t.show()}"
    return None


@dataclass
class Result:
    generated: list[Node]
    promoted: list[tuple[Node, set]]     # (tree, scenarios in which it is profitable)
    pruned: list[tuple[Node, str, str]]  # (tree, reason '>=', reason '<')


def prune(trees: list[Node], attention: bool = False) -> Result:
    promoted, pruned = [], []
    for i, t in enumerate(trees):
        r_ge, r_lt = unprofitable(i, trees, ">=", attention), unprofitable(i, trees, "<", attention)
        if r_ge and r_lt:
            pruned.append((t, r_ge, r_lt))
        else:
            promoted.append((t, {s for s, r in ((">=", r_ge), ("<", r_lt)) if r is None}))
    return Result(trees, promoted, pruned)


def gcn_chain() -> list[Node]:
    """GCN (Eq. 2 L115 after the row-broadcast rewrite of L194): D̃^-1/2 Ã D̃^-1/2 H W"""
    return [_leaf("D", "D"), _leaf("A", "A"), _leaf("D", "D"), _leaf("H", "X", "K1"), _leaf("W", "W")]


def gat_chain() -> list[Node]:
    """GAT (Eq. 5/6 L133-L137): α H W with α the attention's sparse output (Eq. 4)"""
    return [_leaf("α", "S"), _leaf("H", "X", "K1"), _leaf("W", "W")]


GIN_PRE_AGG, GIN_PRE_UPD, GIN_DYN_AGG, GIN_DYN_UPD = 64, 65, 66, 67


def gin_expr() -> list:
    """GIN (reading R23): agg(H) W1 = (Ã + εI) H W1 -- the sum of the sparse pattern and the scaled
    identity, then the dense chain; the MLP's ReLU ends the re-associable part (L192)"""
    return [("+", [_leaf("A", "A")], [_leaf("E", "D")]), _leaf("H", "X", "K1"), _leaf("W", "W")]


def _combine(a: Node, b: Node) -> Node | None:
    """resolve a sum of two associated terms: sparse + diagonal -> SpAdd (sparse values: the
    diagonal folded into Ã, O(nnz)); dense + dense -> Add (element-wise, at their width)"""
    if a.kind in "ASD" and b.kind in "ASD":
        return Node("S", "SpAdd", (a, b), None, "+")
    if a.kind == "X" and b.kind == "X" and a.width == b.width:
        return Node("X", "Add", (a, b), a.width, "+")
    return None


def generate_sum(items: list) -> list[Node]:
    """Algorithm 1 over an IR with sums: besides the adjacent-leaf candidates (rules above), a sum
    factor ("+", P, Q) is either resolved (both terms associated, then combined) or distributed over
    its right neighbour R: (P + Q) R -> P R + Q R.  Returns the de-duplicated forest."""
    out: list[Node] = []
    seen: set = set()

    def resolved(x):
        return isinstance(x, Node)

    def terms(chain):  # every association of a term's chain
        if len(chain) == 1 and resolved(chain[0]):
            return [chain[0]]
        return generate_sum(chain)

    def rec(seq):
        if len(seq) == 1 and resolved(seq[0]):
            key = seq[0].show()
            if key not in seen:
                seen.add(key)
                out.append(seq[0])
            return
        for i, x in enumerate(seq):
            if resolved(x):
                continue
            _, P, Q = x
            for a in terms(P):           # resolve the sum
                for b in terms(Q):
                    n = _combine(a, b)
                    if n is not None:
                        rec(seq[:i] + [n] + seq[i + 1:])
            if i + 1 < len(seq):         # distribute it over its right neighbour
                rec(seq[:i] + [("+", P + [seq[i + 1]], Q + [seq[i + 1]])] + seq[i + 2:])
        plain = [j for j in range(len(seq) - 1) if resolved(seq[j]) and resolved(seq[j + 1])]
        for j in plain:
            for (k0, k, node) in _candidates(seq[j:j + 2]):
                rec(seq[:j] + [node] + seq[j + 2:])

    rec(list(items))
    return out


def composition_id(t: Node) -> int:
    """map a promoted tree to the library's composition id (include/granii.h)"""
    s = t.show()
    table = {
        "((SDDMM(DAD) H) W)": GCN_PRE_AGG, "(SDDMM(DAD) (H W))": GCN_PRE_UPD,
        "((D (A (D H))) W)": GCN_DYN_AGG, "(D (A (D (H W))))": GCN_DYN_UPD,
        "(α (H W))": GAT_REUSE, "((α H) W)": GAT_RECOMP,
        "(((A + E) H) W)": GIN_PRE_AGG, "((A + E) (H W))": GIN_PRE_UPD,
        "(((A H) + (E H)) W)": GIN_DYN_AGG, "((A (H W)) + (E (H W)))": GIN_DYN_UPD,
    }
    return table[s]


def evaluate(t: Node, env: dict):
    """dense value of a tree, leaves looked up by name in env (numpy / torch matrices): the
    semantic-equivalence check of L192 (every re-association computes the same product)"""
    if t.prim == "SDDMM" and not t.kids:
        return env["D"] @ env["A"] @ env["D"]
    if not t.kids:
        return env[t.name]
    if t.prim in ("SpAdd", "Add"):
        return evaluate(t.kids[0], env) + evaluate(t.kids[1], env)
    v = evaluate(t.kids[0], env)
    for k in t.kids[1:]:
        v = v @ evaluate(k, env)
    return v


def forest(model: str) -> list[Node]:
    if model == "gin":
        return generate_sum(gin_expr())
    return generate(gcn_chain() if model == "gcn" else gat_chain())


def promoted_compositions(model: str) -> dict[int, set]:
    """{composition id: scenarios in which it is promoted} for 'gcn', 'gat' or 'gin' (GIN's
    scenarios compare K1 with the MLP's hidden width Kh, the width its aggregation runs at)"""
    res = prune(forest(model), attention=model == "gat")
    return {composition_id(t): sc for t, sc in res.promoted}


if __name__ == "__main__":
    for m in ("GCN", "GAT", "GIN"):
        r = prune(forest(m.lower()), attention=m == "GAT")
        print(f"{m}: {len(r.generated)} generated, {len(r.pruned)} pruned, {len(r.promoted)} promoted")
        for t, sc in r.promoted:
            print("  promoted", t.show(), sorted(sc), "->", composition_id(t))
        for t, a, b in r.pruned:
            print("  pruned  ", t.show(), "|", a, "|", b)
