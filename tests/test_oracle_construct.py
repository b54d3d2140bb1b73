"""Pins for the oracle's token-tree construction (NEXT-2, §3):
expansion by a static configuration <k1..km> (Fig. 3), top-k expansion of SSM outputs,
depth-first linearisation (Fig. 2) and token tree merge (Def. 3.2; Fig. 2).

Independent of the oracle's code: the figures' worked examples (golden files), the closed-form
node count 1 + sum_i prod_{j<=i} k_j, Def. 3.2's defining property checked by brute-force
enumeration of the sequence sets S_u (Def. 3.1), and numpy's stable argsort for top-k."""
import itertools

import numpy as np
import pytest

import oracle
import workloads as W
from tests.conftest import load_golden


def _seqs(parent, tokens):
    """The set {S_u} of Def. 3.1 (L450-454) by brute force."""
    out = set()
    for u in range(len(parent)):
        s, x = [], u
        while x >= 0:
            s.append(int(tokens[x]))
            x = parent[x]
        out.add(tuple(s[::-1]))
    return out


def test_fig3_expansion_topology_and_sequences():
    g = load_golden("fig3_expansion.json")
    par, dep = oracle.expansion_tree_bfs(g["expansion"])
    assert len(par) == g["n_nodes"]
    dpar, _, order = oracle.dfs_linearize(par)
    assert dpar == g["dfs_parent"]
    # the figure's tokens: expand each frontier node by its listed top-k tokens, step by step
    steps = g["tokens_by_step"]
    tok = {0: steps["root"]}
    for u in range(1, len(par)):
        p = par[u]
        sibs = [c for c in range(1, len(par)) if par[c] == p]
        tok[u] = steps[str(dep[u] - 1)][tok[p]][sibs.index(u)]
    leaves = [u for u in range(len(par)) if u not in par]
    got = []
    for leaf in leaves:
        s, x = [], leaf
        while x >= 0:
            s.append(tok[x])
            x = par[x]
        got.append(s[::-1])
    assert sorted(map(tuple, got)) == sorted(map(tuple, g["sequences"]))
    assert len(leaves) == g["n_leaves"]


def test_expansion_node_count_closed_form():
    rng = np.random.default_rng(0)
    for _ in range(100):
        ks = [int(x) for x in rng.integers(1, 5, int(rng.integers(0, 6)))]
        par, dep = oracle.expansion_tree_bfs(ks)
        assert len(par) == 1 + sum(int(np.prod(ks[:i + 1])) for i in range(len(ks)))
        assert max(dep) == len(ks)
        dpar, _, _ = oracle.dfs_linearize(par)
        # same tree as the (independently written) input generator's DFS expansion tree
        assert dpar == list(W.expansion_tree(ks)[0])


def test_expand_topk_against_stable_argsort():
    rng = np.random.default_rng(1)
    for _ in range(50):
        V = int(rng.integers(2, 200))
        row = rng.integers(-3, 3, V).astype(np.float32)  # many ties
        k = int(rng.integers(1, min(V, 8) + 1))
        ref = np.argsort(-row.astype(np.float64), kind="stable")[:k]
        assert oracle.expand_topk(row, k) == list(ref)


def test_fig2_merge():
    g = load_golden("fig2_merge.json")
    vocab = sorted({w for s in g["inputs"] for w in s})
    ids = {w: i for i, w in enumerate(vocab)}
    trees = [(list(range(-1, len(s) - 1)), [ids[w] for w in s]) for s in g["inputs"]]
    par, tok, dep, maps = oracle.tree_merge(trees)
    assert par == g["merged_parent"]
    assert [vocab[t] for t in tok] == g["merged_tokens"]
    assert dep == [0, 1, 2, 2, 3, 1, 2]
    # every input node (the inputs are chains) maps to the merged node with the same sequence
    for (ip, it), m in zip(trees, maps):
        for i in range(len(ip)):
            s = []
            x = m[i]
            while x >= 0:
                s.append(tok[x])
                x = par[x]
            assert tuple(s[::-1]) == tuple(it[:i + 1])


def test_merge_definition_3_2_brute_force():
    """Def. 3.2: M is the merge of {N_i} iff every S_u of every input has an S_v in M and vice
    versa; a merge has no two siblings with the same token (each sequence is one node)."""
    rng = np.random.default_rng(2)
    for _ in range(100):
        T = int(rng.integers(1, 5))
        trees = []
        for _ in range(T):
            n = int(rng.integers(1, 12))
            par, _ = W.random_tree(n, 6, 3, rng)
            tok = rng.integers(0, 3, n).astype(int)
            tok[0] = 7
            trees.append((list(par), list(tok)))
        par, tok, dep, maps = oracle.tree_merge(trees)
        union = set().union(*[_seqs(p, t) for p, t in trees])
        assert _seqs(par, tok) == union
        assert len(par) == len(union)
        for u, v in itertools.combinations(range(len(par)), 2):
            assert not (par[u] == par[v] and tok[u] == tok[v])
        assert all(par[i] < i for i in range(1, len(par))) and par[0] == -1
    # roots must agree
    assert oracle.tree_merge([([-1], [1]), ([-1], [2])]) is None


def test_ssm_distribution_pins():
    """The draft row (R12) against a library routine (scipy softmax of logits / T), a closed form
    (two tokens: p0 = 1 / (1 + e^{(l1 - l0) / T})) and the T -> 0 / uniform special cases."""
    from scipy.special import softmax
    rng = np.random.default_rng(3)
    for T in (0.5, 1.0, 1.7):
        row = rng.normal(size=97).astype(np.float32) * 3
        np.testing.assert_allclose(oracle.ssm_distribution(row, T), softmax(row.astype(np.float64) / T),
                                   rtol=1e-12, atol=0)
    q = oracle.ssm_distribution(np.array([1.0, -0.5], np.float32), 0.8)
    assert q[0] == pytest.approx(1.0 / (1.0 + np.exp((-0.5 - 1.0) / 0.8)), rel=1e-14)
    assert np.array_equal(oracle.ssm_distribution(np.zeros(8, np.float32)), np.full(8, 1 / 8))
    assert oracle.ssm_distribution(np.array([2.0, 1.0], np.float32), 1e-3)[0] == 1.0


def test_validate_tree_every_branch():
    """Def. 3.1 (L450-454) validity, one defect at a time on the Fig. 4 tree (golden): n_nodes out
    of [1, Nmax], P + n > Smax, a root with a parent, a parent not before its child, depth not
    parent's + 1, depth beyond Dmax; the valid tree passes at exactly the limits."""
    g = load_golden("fig4_mask.json")
    par = np.asarray(g["parent"], np.int32)
    n = len(par)
    dep = np.zeros(n, np.int32)
    for i in range(1, n):
        dep[i] = dep[par[i]] + 1
    D = int(dep.max())
    ok = lambda p, d, P=5, nn=n, nmax=n, dmax=D, smax=5 + n: oracle.validate_tree(p, d, P, nn, nmax, dmax, smax)
    assert ok(par, dep) == 0
    assert ok(par, dep, nn=0) != 0 and ok(par, dep, nn=n + 1) != 0            # n_nodes range
    assert ok(par, dep, smax=5 + n - 1) != 0 and ok(par, dep, P=-1) != 0      # P + n > Smax, P < 0
    p2 = par.copy(); p2[0] = 0
    assert ok(p2, dep) != 0                                                   # root has a parent
    p3 = par.copy(); p3[3] = 5
    assert ok(p3, dep) != 0                                                   # parent after child
    d2 = dep.copy(); d2[4] += 1
    assert ok(par, d2) != 0                                                   # depth != depth[parent] + 1
    assert ok(par, dep, dmax=D - 1) != 0                                      # depth > Dmax
    assert ok(par, None, dmax=0) == 0                                         # no depth array: topology only
