"""Pins for the oracle's tree -> sequences decomposition (NEXT-1, sequence-based decoding,
PAPER.md §4.2, Fig. 4 left L682) and for the claim that sequence-based decoding
computes the same attention outputs as tree-based decoding (L671-673).

Independent of the oracle's code: the Fig. 4 worked example (three kernels, 13 query rows),
brute-force enumeration of root-to-leaf paths over the explicit sequence sets S_u (Def. 3.1), and
the oracle's own tree attention checked against per-sequence causal attention computed with
torch SDPA in float64.
"""
import itertools

import numpy as np
import torch

import oracle
import workloads as W
from tests.conftest import load_golden


def test_fig4_sequences():
    """Fig. 4 (L682): the tree decomposes into Kernel 1 (t2 t3 t4 t5), Kernel 2 (t2 t3 t8 t9) and
    Kernel 3 (t2 t3 t4 t6 t7): 3 sequences, 13 query rows."""
    g = load_golden("fig4_mask.json")
    parent = np.asarray([g["parent"]], np.int32)
    paths = oracle.leaf_paths(parent, [len(g["parent"])])[0]
    names = [[g["nodes"][i] for i in p] for p in paths]
    assert sorted(map(tuple, names)) == sorted(map(tuple, g["sequences"]))
    assert sum(len(p) for p in paths) == g["sequence_query_rows"]
    # node-index order of the leaves is the DFS order of the linearised tree (t5, t7, t9)
    assert [p[-1] for p in paths] == [3, 5, 7]


def _sequences_by_definition(par):
    """Def. 3.1 / 3.2 (L450-454, L519-527): every node u has the sequence S_u; the tree's token
    sequences are the maximal ones, i.e. those S_u that are not a proper prefix of another S_v."""
    n = len(par)
    seqs = []
    for u in range(n):
        s, x = [], u
        while x >= 0:
            s.append(x)
            x = par[x]
        seqs.append(tuple(s[::-1]))
    return sorted(s for s in seqs if not any(len(t) > len(s) and t[:len(s)] == s for t in seqs))


def test_leaf_paths_brute_force_random_trees():
    rng = np.random.default_rng(7)
    for _ in range(200):
        n = int(rng.integers(1, 40))
        par, _ = W.random_tree(n, 8, 4, rng)
        got = oracle.leaf_paths(np.asarray([par], np.int32), [n])[0]
        assert sorted(map(tuple, got)) == _sequences_by_definition(list(par))
        # every node lies on at least one sequence; leaves are exactly the sequence ends
        assert set(itertools.chain.from_iterable(got)) == set(range(n))


def test_leaf_paths_invalid_and_degenerate():
    assert oracle.leaf_paths(np.asarray([[-1, 0, 5]], np.int32), [3]) == [None]
    assert oracle.leaf_paths(np.asarray([[0, 0]], np.int32), [2]) == [None]
    assert oracle.leaf_paths(np.asarray([[-1]], np.int32), [1]) == [[[0]]]          # root only
    chain = W.chain_tree(5)[0]
    assert oracle.leaf_paths(np.asarray([chain], np.int32), [5]) == [[[0, 1, 2, 3, 4]]]


def test_tree_attention_equals_sequence_decoding():
    """L671-673: tree attention "computes the exact same attention output" as decoding each
    sequence separately with its own KV cache (Fig. 4 left): per sequence, causal SDPA (float64)
    over [prefix, sequence tokens] reproduces the oracle's tree output at every node on it."""
    rng = np.random.default_rng(3)
    n, P, H = 12, 5, 2
    par, dep = W.random_tree(n, 4, 3, rng)
    tb = W.make_tree_batch([(par, dep)], [P])
    q = W.randn_bf16((1, n, H, 128), 11)
    k = W.randn_bf16((1, H, P + n, 128), 12)
    v = W.randn_bf16((1, H, P + n, 128), 13)
    tree = oracle.tree_attention(q, k, v, tb.parent, tb.depth, tb.prefix_len, tb.n_nodes)
    for path in oracle.leaf_paths(tb.parent.numpy(), tb.n_nodes.numpy())[0]:
        slots = list(range(P)) + [P + j for j in path]
        for h in range(H):
            kk = k[0, h, slots].to(torch.float64)
            vv = v[0, h, slots].to(torch.float64)
            qq = q[0, path, h].to(torch.float64)
            L = len(path)
            mask = torch.ones((L, P + L), dtype=torch.bool)
            mask[:, P:] = torch.tril(torch.ones((L, L), dtype=torch.bool))
            ref = torch.nn.functional.scaled_dot_product_attention(qq[None], kk[None], vv[None], attn_mask=mask,
                                                                   scale=128 ** -0.5)[0]
            np.testing.assert_allclose(tree[0, path, h], ref.numpy(), atol=1e-10, rtol=0)
