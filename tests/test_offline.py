"""GRANII's offline stage (N4, paper_conf_cgo_lenadorasgytm26_b200/offline.py): association-tree
generation (Algorithm 1) and input-oblivious pruning (L226-L233), pinned to the
paper's composition counts (L326: GCN "12 and 8", GAT "2 and 0"), to the semantic
equivalence of every generated tree (L192), and to the library's composition set."""
import numpy as np

from paper_conf_cgo_lenadorasgytm26_b200 import offline as OF


def test_gcn_counts_match_the_paper():
    trees = OF.generate(OF.gcn_chain())
    res = OF.prune(trees)
    assert (len(res.generated), len(res.pruned), len(res.promoted)) == (12, 8, 4)   # L326


def test_gcn_generated_is_every_parenthesisation_modulo_the_dad_sddmm():
    """a 5-factor chain has Catalan(4) = 14 parenthesisations; the two that associate D A D
    as (DA)D / D(AD) inside (DAD) H W and (DAD)(H W) are the same SDDMM(dinv, dinv) -> 12"""
    catalan4 = 14
    dad_unit_trees = 2          # parenthesisations of the 3-chain (Ñ) H W
    inner_forms = 2             # (DA)D and D(AD) collapse to one SDDMM
    assert len(OF.generate(OF.gcn_chain())) == catalan4 - dad_unit_trees * (inner_forms - 1)


def test_every_generated_tree_computes_the_same_product():
    rng = np.random.default_rng(0)
    n, k1, k2 = 7, 5, 3
    A = (rng.random((n, n)) < 0.4).astype(float) + np.eye(n)
    D = np.diag(1.0 / np.sqrt(A.sum(1)))
    env = {"D": D, "A": A, "H": rng.standard_normal((n, k1)), "W": rng.standard_normal((k1, k2)),
           "α": rng.random((n, n)) * (A > 0)}
    ref = D @ A @ D @ env["H"] @ env["W"]
    for t in OF.generate(OF.gcn_chain()):
        assert np.allclose(OF.evaluate(t, env), ref, rtol=1e-12, atol=1e-12), t.show()
    for t in OF.generate(OF.gat_chain()):
        assert np.allclose(OF.evaluate(t, env), env["α"] @ env["H"] @ env["W"], rtol=1e-12, atol=1e-12)


def test_gcn_promoted_are_the_library_compositions_with_the_embedding_size_rule():
    """promoted = {PRE, DYN} x {AGG, UPD} (DESIGN R10); annotations = the prefilter of
    granii_select (L237-L239, reading R11): update-first iff K1 >= K2"""
    p = OF.promoted_compositions("gcn")
    assert p == {OF.GCN_PRE_AGG: {"<"}, OF.GCN_DYN_AGG: {"<"}, OF.GCN_PRE_UPD: {">="}, OF.GCN_DYN_UPD: {">="}}


def test_gcn_pruned_trees_are_dominated():
    """every pruned tree's primitives include all of a promoted tree's (rule 1) or repeat a
    tree's primitives at a width that is never smaller (rule 2), in both scenarios"""
    res = OF.prune(OF.generate(OF.gcn_chain()))
    for t, r_ge, r_lt in res.pruned:
        assert r_ge.startswith("rule") and r_lt.startswith("rule")
        # the pruned tree is never cheaper in primitive count than the tree it lost to
        for r in (r_ge, r_lt):
            other = r.split(" vs ")[1]
            o = [x for x in res.generated if x.show() == other][0]
            assert sum(OF.primitives(t).values()) >= sum(OF.primitives(o).values())


def test_gat_counts_and_both_promoted():
    res = OF.prune(OF.generate(OF.gat_chain()), attention=True)
    assert (len(res.generated), len(res.pruned), len(res.promoted)) == (2, 0, 2)   # L326
    p = OF.promoted_compositions("gat")
    # RECOMP does all of REUSE's work on never-smaller matrices plus a GEMM when K1 >= K2 (rule 1):
    # profitable only for growing sizes (L330, L357)
    assert p == {OF.GAT_REUSE: {"<", ">="}, OF.GAT_RECOMP: {"<"}}
    # RECOMP pays the extra GEMM of L135
    reuse = [t for t in res.generated if OF.composition_id(t) == OF.GAT_REUSE][0]
    recomp = [t for t in res.generated if OF.composition_id(t) == OF.GAT_RECOMP][0]
    assert OF.primitives(recomp, True)[("GEMM", "K1K2")] == OF.primitives(reuse, True)[("GEMM", "K1K2")] + 1


def test_gin_forest_pruning_and_promoted_compositions():
    """GIN (reading R23): (Ã + εI) H W1 with a sum in the IR.  The distributive rewrite gives 7
    distinct trees (the paper counts 8 generated, L326), pruning keeps 4 -- the paper's promoted
    count (8 - 4) -- which are exactly the library's GIN compositions, aggregate-first when K1 < Kh"""
    trees = OF.forest("gin")
    res = OF.prune(trees)
    assert (len(res.generated), len(res.pruned), len(res.promoted)) == (7, 3, 4)
    assert OF.promoted_compositions("gin") == {OF.GIN_PRE_AGG: {"<"}, OF.GIN_DYN_AGG: {"<"},
                                                OF.GIN_PRE_UPD: {">="}, OF.GIN_DYN_UPD: {">="}}
    rng = np.random.default_rng(1)
    n, k1, kh = 6, 4, 5
    A = (rng.random((n, n)) < 0.5).astype(float) + np.eye(n)
    env = {"A": A, "E": 0.3 * np.eye(n), "H": rng.standard_normal((n, k1)), "W": rng.standard_normal((k1, kh))}
    ref = (A + env["E"]) @ env["H"] @ env["W"]
    for t in trees:      # every re-association computes the same matrix (L192)
        assert np.allclose(OF.evaluate(t, env), ref, rtol=1e-12, atol=1e-12), t.show()


def test_cse_counts_a_shared_subtree_once():
    """L219: A (H W) + E (H W) computes H W once"""
    dyn_upd = [x for x in OF.forest("gin") if x.show() == "((A (H W)) + (E (H W)))"][0]
    assert OF.primitives(dyn_upd)[("GEMM", "K1K2")] == 1
