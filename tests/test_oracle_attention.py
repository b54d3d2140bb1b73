"""Pins for the oracle's tree attention (oracle/ c1) against what the paper and mathematics fix.

Each test is independent of the oracle's code: it uses a worked example from the paper, a
closed form, a textbook/library routine (torch SDPA in float64), brute force over explicit
sequences S_u, or an invariant.  Citations are PAPER.md line numbers.
"""
import numpy as np
import pytest
import torch

import oracle
import workloads as W
from tests.conftest import load_golden

D = 128


def _bf16(a):
    return torch.as_tensor(a, dtype=torch.float32).to(torch.bfloat16)


def _f64(t):
    return t.to(torch.float64)


def _rand_inputs(B, Nmax, Hq, Hkv, Smax, seed, scale=1.0):
    q = W.randn_bf16((B, Nmax, Hq, D), seed, scale=scale)
    k = W.randn_bf16((B, Hkv, Smax, D), seed + 1)
    v = W.randn_bf16((B, Hkv, Smax, D), seed + 2)
    return q, k, v


def _path(parent, i):
    """S_u by Def. 3.1 (L450-454): S_u = S_{p_u} + t_u, built recursively from the root."""
    if i < 0:
        return []
    return _path(parent, int(parent[i])) + [i]


def _seq_attention_last(qrow, keys, vals, scale):
    """Original sequence attention (Eq. 1-3) for the LAST token of a sequence:
    torch SDPA in float64 (library routine)."""
    qq = _f64(qrow)[None, None, None, :]
    kk = _f64(keys)[None, None]
    vv = _f64(vals)[None, None]
    return torch.nn.functional.scaled_dot_product_attention(qq, kk, vv, scale=scale)[0, 0, 0]


def test_fig4_topology_aware_mask():
    """Fig. 4 (L682): key-column tick counts [8,7,4,1,2,1,2,1], 26 visible pairs.

    With P = 0, all keys equal (uniform weights over visible keys) and V_j = e_j, out[i][j] =
    1/|Anc*(i)| iff key j is visible to node i, so the oracle's visibility can be read off."""
    g = load_golden("fig4_mask.json")
    parent = np.asarray(g["parent"], np.int32)
    n = len(parent)
    q = _bf16(np.random.default_rng(0).standard_normal((1, n, 1, D)))
    k = torch.zeros((1, 1, n, D), dtype=torch.bfloat16)
    v = torch.zeros((1, 1, n, D), dtype=torch.bfloat16)
    for j in range(n):
        v[0, 0, j, j] = 1.0
    out = oracle.tree_attention(q, k, v, parent[None], None, [0], [n])
    vis = out[0, :, 0, :n] > 0
    assert vis.sum(axis=0).tolist() == g["column_tick_counts"]
    assert int(vis.sum()) == g["total_visible_pairs"]
    # each row's weights are exactly uniform over its visible keys (mask = exactly 0 weight, L627-628)
    for i in range(n):
        cnt = vis[i].sum()
        assert np.all(out[0, i, 0, :n][vis[i]] == pytest.approx(1.0 / cnt, abs=0, rel=1e-15))
        assert np.all(out[0, i, 0, :n][~vis[i]] == 0.0)
    # the three root-to-leaf sequences of sequence-based decoding cover 13 query rows
    leaves = [i for i in range(n) if i not in set(parent.tolist())]
    seqs = [_path(parent, l) for l in leaves]
    names = g["nodes"]
    assert sorted([[names[i] for i in s] for s in seqs]) == sorted(g["sequences"])
    assert sum(len(s) for s in seqs) == g["sequence_query_rows"]


@pytest.mark.parametrize("P,n", [(0, 1), (5, 1), (17, 9), (64, 33)])
def test_chain_equals_causal_incremental_decoding(P, n):
    """A chain tree is ordinary causal decoding (Eq. 4; 'exact same attention output
    as incremental decoding', L671-673): row i = decode attention over P + i + 1 keys."""
    Hq = Hkv = 2
    Smax = P + n + 3
    q, k, v = _rand_inputs(1, n, Hq, Hkv, Smax, 11)
    parent, depth = W.chain_tree(n)
    out = oracle.tree_attention(q, k, v, parent[None], depth[None], [P], [n])
    scale = 1.0 / np.sqrt(D)
    # independent causal attention: scores over the whole sequence with a lower-triangular mask
    for h in range(Hq):
        Q = _f64(q[0, :, h])                        # [n][D] queries at positions P..P+n-1
        K = _f64(k[0, h, :P + n])
        V = _f64(v[0, h, :P + n])
        S = (Q @ K.T) * scale                       # [n][P+n]
        pos_q = torch.arange(P, P + n)[:, None]
        pos_k = torch.arange(P + n)[None, :]
        S = S.masked_fill(pos_k > pos_q, float("-inf"))
        ref = torch.softmax(S, dim=-1) @ V
        np.testing.assert_allclose(out[0, :, h], ref.numpy(), rtol=1e-12, atol=1e-12)


def test_per_node_bruteforce_sequences():
    """Def. 4.1 (L594-598): TreeAttention(u) = Attention(S_u).  For every node, build S_u
    explicitly (committed prefix + its root path) and run plain sequence attention."""
    rng = np.random.default_rng(3)
    B, Hq, Hkv, Nmax = 3, 4, 2, 16
    trees = [W.random_tree(int(rng.integers(1, Nmax + 1)), 6, 3, rng) for _ in range(B)]
    P = [0, 7, 30]
    tb = W.make_tree_batch(trees, P, max_nodes=Nmax)
    Smax = max(P) + Nmax
    q, k, v = _rand_inputs(B, Nmax, Hq, Hkv, Smax, 21, scale=2.0)
    out = oracle.tree_attention(q, k, v, tb.parent, tb.depth, tb.prefix_len, tb.n_nodes)
    scale = 1.0 / np.sqrt(D)
    G = Hq // Hkv
    for b in range(B):
        par = tb.parent[b].numpy()
        for i in range(int(tb.n_nodes[b])):
            slots = list(range(P[b])) + [P[b] + j for j in _path(par, i)]
            for h in range(Hq):
                ref = _seq_attention_last(q[b, i, h], k[b, h // G, slots], v[b, h // G, slots], scale)
                np.testing.assert_allclose(out[b, i, h], ref.numpy(), rtol=1e-11, atol=1e-12)


def test_against_sdpa_with_explicit_mask_gqa():
    """Library routine: torch SDPA (float64) with the explicit boolean mask
    [prefix all-true | ancestor-or-self matrix] and GQA head mapping g = h // (Hq/Hkv)."""
    rng = np.random.default_rng(5)
    B, Hq, Hkv, Nmax, P = 2, 8, 2, 12, 9
    trees = [W.random_tree(Nmax, 5, 4, rng), W.random_tree(5, 5, 4, rng)]
    tb = W.make_tree_batch(trees, [P, P], max_nodes=Nmax)
    Smax = P + Nmax + 1
    q, k, v = _rand_inputs(B, Nmax, Hq, Hkv, Smax, 31)
    out = oracle.tree_attention(q, k, v, tb.parent, tb.depth, tb.prefix_len, tb.n_nodes)
    for b in range(B):
        n = int(tb.n_nodes[b])
        par = tb.parent[b].numpy()
        mask = torch.zeros((n, P + n), dtype=torch.bool)
        mask[:, :P] = True
        for i in range(n):
            u = i
            while u >= 0:
                mask[i, P + u] = True
                u = int(par[u])
        Q = _f64(q[b, :n]).permute(1, 0, 2)                         # [Hq][n][D]
        K = _f64(k[b, :, :P + n]).repeat_interleave(Hq // Hkv, 0)   # [Hq][P+n][D]
        V = _f64(v[b, :, :P + n]).repeat_interleave(Hq // Hkv, 0)
        ref = torch.nn.functional.scaled_dot_product_attention(Q, K, V, attn_mask=mask)
        np.testing.assert_allclose(out[b, :n], ref.permute(1, 0, 2).numpy(), rtol=1e-11, atol=1e-12)
        assert np.all(np.isnan(out[b, n:]))   # padded rows untouched


def test_closed_forms():
    """Eq. 3 (L566) closed forms: (a) all visible keys equal => out = mean of visible V;
    (b) P = 0 and a root-only tree => out = v_root exactly."""
    rng = np.random.default_rng(7)
    n, P = 7, 5
    parent, depth = W.random_tree(n, 4, 3, rng)
    q = W.randn_bf16((1, n, 1, D), 41)
    k = torch.zeros((1, 1, P + n, D), dtype=torch.bfloat16)
    k[:] = W.randn_bf16((D,), 42)
    v = W.randn_bf16((1, 1, P + n, D), 43)
    out = oracle.tree_attention(q, k, v, parent[None], depth[None], [P], [n])
    for i in range(n):
        slots = list(range(P)) + [P + j for j in _path(parent, i)]
        ref = _f64(v[0, 0, slots]).mean(0).numpy()
        np.testing.assert_allclose(out[0, i, 0], ref, rtol=1e-12, atol=1e-14)
    out1 = oracle.tree_attention(q[:, :1], k, v, np.array([[-1]]), np.array([[0]]), [0], [1])
    assert np.array_equal(out1[0, 0, 0], _f64(v[0, 0, 0]).numpy())


def test_topological_reorder_invariance():
    """The node order is a storage choice (tree topology in the KV cache, L659-661): any
    topological re-ordering of the nodes (with their q/K/V) permutes the outputs."""
    rng = np.random.default_rng(9)
    n, P, Hq = 14, 6, 2
    parent, depth = W.random_tree(n, 5, 3, rng)
    q, k, v = _rand_inputs(1, n, Hq, Hq, P + n, 51)
    out = oracle.tree_attention(q, k, v, parent[None], depth[None], [P], [n])
    # BFS order is another topological order
    order = sorted(range(n), key=lambda i: (depth[i], i))
    new_of = {old: new for new, old in enumerate(order)}
    par2 = np.asarray([-1 if parent[o] < 0 else new_of[int(parent[o])] for o in order], np.int32)
    dep2 = depth[order]
    q2 = q[:, order]
    k2 = k.clone()
    v2 = v.clone()
    k2[:, :, P:P + n] = k[:, :, [P + o for o in order]]
    v2[:, :, P:P + n] = v[:, :, [P + o for o in order]]
    out2 = oracle.tree_attention(q2, k2, v2, par2[None], dep2[None], [P], [n])
    np.testing.assert_allclose(out2[0], out[0, order], rtol=1e-13, atol=1e-15)


def test_invalid_trees_untouched():
    """Tree defects (parent not < i, depth mismatch, P + n > Smax) produce no output."""
    q, k, v = _rand_inputs(1, 4, 1, 1, 8, 61)
    bad = [
        (np.array([[-1, 0, 3, 1]]), np.array([[0, 1, 2, 2]]), 2, 4),   # parent[2] = 3 >= 2
        (np.array([[-1, 0, 1, 1]]), np.array([[0, 1, 2, 3]]), 2, 4),   # depth mismatch
        (np.array([[-1, 0, 1, 1]]), np.array([[0, 1, 2, 2]]), 6, 4),   # P + n > Smax
        (np.array([[0, 0, 1, 1]]), np.array([[0, 1, 2, 2]]), 2, 4),    # root has a parent
    ]
    for parent, depth, P, n in bad:
        out = oracle.tree_attention(q, k, v, parent, depth, [P], [n])
        assert np.all(np.isnan(out))
