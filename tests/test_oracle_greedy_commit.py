"""Pins for the oracle's greedy verification (c3) and depth-first KV-cache commit (c2)."""
import itertools

import numpy as np
import pytest
import torch

import oracle
import workloads as W
from tests.conftest import load_golden

D = 128


def _onehot_logits(B, Nmax, V, argmax_tokens):
    """Logits whose unique argmax per node is the given token (others strictly smaller)."""
    rng = np.random.default_rng(0)
    lg = rng.uniform(-1, 0, size=(B, Nmax, V)).astype(np.float32)
    for b in range(B):
        for u, t in enumerate(argmax_tokens[b]):
            lg[b, u, t] = 5.0
    return lg


def test_fig2_worked_example():
    """Fig. 2 (L304-317): LLM outputs [learning, system, design, optimization, EOS, model, EOS]
    over the DFS-linearised tree give 'machine learning system optimization' (L313)."""
    g = load_golden("fig2_greedy.json")
    vocab = {w: i for i, w in enumerate(g["vocab"])}
    toks = np.asarray([[vocab[w] for w in g["tree_tokens"]]], np.int32)
    parent = np.asarray([g["parent"]], np.int32)
    outs = [[vocab[w] for w in g["llm_output"]]]
    n = toks.shape[1]
    lg = _onehot_logits(1, n, len(vocab), outs)
    an, at, na = oracle.verify_greedy(lg, toks, parent, [n])
    assert na[0] == len(g["expected_accepted_nodes"])
    assert an[0, :na[0]].tolist() == g["expected_accepted_nodes"]
    words = [g["vocab"][t] for t in at[0, :na[0]]]
    assert words == g["expected_tokens"]
    assert " ".join([g["tree_tokens"][0]] + words) == g["expected_text"]
    assert np.all(an[0, na[0]:] == -1) and np.all(at[0, na[0]:] == -1)


def test_fig2_commit_moves_node3_to_slot_P_plus_2():
    """DFS KV update (L635-644) for the Fig. 2 path [0,1,3]: slots P, P+1 keep their rows,
    slot P+2 receives node 3's row, P advances by 3."""
    L, B, Hkv, Smax, P = 2, 1, 3, 16, 5
    k = W.randn_bf16((L, B, Hkv, Smax, D), 71).view(torch.int16).numpy().view(np.uint16).copy()
    v = W.randn_bf16((L, B, Hkv, Smax, D), 72).view(torch.int16).numpy().view(np.uint16).copy()
    k0, v0 = k.copy(), v.copy()
    pl = np.array([P], np.int32)
    oracle.kv_commit(k, v, pl, np.array([[0, 1, 3, -1]], np.int32), np.array([3], np.int32))
    assert pl[0] == P + 3
    for a, a0 in ((k, k0), (v, v0)):
        assert np.array_equal(a[..., :P + 2, :], a0[..., :P + 2, :])
        assert np.array_equal(a[..., P + 2, :], a0[..., P + 3, :])


def test_commit_identity_path_is_noop():
    """The leftmost DFS branch is stored in place (path[j] = j): committing it changes nothing
    but P (the DFS layout of L638-644)."""
    L, B, Hkv, Smax, P = 1, 2, 2, 20, 4
    k = np.random.default_rng(1).integers(0, 2**16, (L, B, Hkv, Smax, D), dtype=np.uint16)
    v = k[::-1].copy()
    k0, v0 = k.copy(), v.copy()
    pl = np.array([P, P + 1], np.int32)
    path = np.array([[0, 1, 2, 3, 4], [0, 1, -1, -1, -1]], np.int32)
    oracle.kv_commit(k, v, pl, path, np.array([5, 2], np.int32))
    assert np.array_equal(k, k0) and np.array_equal(v, v0)
    assert pl.tolist() == [P + 5, P + 3]


def test_commit_then_root_only_equals_chain_attention():
    """After commit (L635-644), the next iteration's root-only tree over the new cache equals
    plain sequence attention over prefix + the accepted tokens' K/V + the new root: the cache
    is what incremental decoding of the accepted tokens would have produced (L671-673)."""
    rng = np.random.default_rng(2)
    n, P, Hq = 12, 9, 2
    parent, depth = W.random_tree(n, 5, 3, rng)
    # pick a random root-to-leaf path
    leaf = int(rng.choice([i for i in range(n) if i not in set(parent.tolist())]))
    path = []
    u = leaf
    while u >= 0:
        path.append(u)
        u = int(parent[u])
    path = path[::-1]
    Smax = P + n + 4
    kt = W.randn_bf16((1, 1, Hq, Smax, D), 81)
    vt = W.randn_bf16((1, 1, Hq, Smax, D), 82)
    k = kt.view(torch.int16).numpy().view(np.uint16).copy()
    v = vt.view(torch.int16).numpy().view(np.uint16).copy()
    pl = np.array([P], np.int32)
    oracle.kv_commit(k, v, pl, np.array([path], np.int32), np.array([len(path)], np.int32))
    Pn = int(pl[0])
    assert Pn == P + len(path)
    q = W.randn_bf16((1, 1, Hq, D), 83)
    kk = torch.from_numpy(k[0].view(np.int16)).view(torch.bfloat16)
    vv = torch.from_numpy(v[0].view(np.int16)).view(torch.bfloat16)
    out = oracle.tree_attention(q, kk, vv, np.array([[-1]]), np.array([[0]]), [Pn], [1])
    # reference: sequence = original prefix rows, original rows of the path nodes, new root row
    slots = list(range(P)) + [P + j for j in path]
    for h in range(Hq):
        keys = torch.cat([kt[0, 0, h, slots], kk[0, h, Pn:Pn + 1]]).to(torch.float64)
        vals = torch.cat([vt[0, 0, h, slots], vv[0, h, Pn:Pn + 1]]).to(torch.float64)
        ref = torch.softmax(keys @ q[0, 0, h].to(torch.float64) / np.sqrt(D), 0) @ vals
        np.testing.assert_allclose(out[0, 0, h], ref.numpy(), rtol=1e-12, atol=1e-13)


def test_greedy_root_only_and_chain():
    """A root-only tree is incremental decoding: exactly one token, the argmax (L980-983).
    A chain is sequence-based speculation: the longest draft prefix that equals the argmaxes."""
    rng = np.random.default_rng(3)
    V = 50
    lg = rng.standard_normal((1, 1, V)).astype(np.float32)
    an, at, na = oracle.verify_greedy(lg, np.zeros((1, 1), np.int32), np.array([[-1]]), [1])
    assert na[0] == 1 and an[0, 0] == 0 and at[0, 0] == int(np.argmax(lg[0, 0]))
    n = 9
    parent, _ = W.chain_tree(n)
    for match in range(n):
        lg = rng.standard_normal((1, n, V)).astype(np.float32)
        am = lg[0].argmax(-1)
        toks = np.zeros((1, n), np.int32)
        for c in range(1, n):
            toks[0, c] = am[c - 1] if c <= match else (am[c - 1] + 1) % V
        an, at, na = oracle.verify_greedy(lg, toks, parent[None], [n])
        assert na[0] == match + 1
        assert an[0, :na[0]].tolist() == list(range(match + 1))
        assert at[0, :match].tolist() == toks[0, 1:match + 1].tolist()
        assert at[0, match] == am[match]


def test_greedy_bruteforce_longest_matching_path():
    """Enumerate every root path, keep the fully matching ones (each child's token equals the
    LLM argmax at its parent, L704-713), take the longest; then append the argmax at its end."""
    rng = np.random.default_rng(4)
    V = 6   # small vocab => many matches
    for trial in range(200):
        n = int(rng.integers(1, 20))
        parent, _ = W.random_tree(n, 6, 3, rng)
        # distinct sibling tokens (Def. 3.2 merged trees have unique sequences, L519-527)
        toks = np.zeros(n, np.int32)
        kids = {}
        for c in range(1, n):
            kids.setdefault(int(parent[c]), []).append(c)
        for u, cs in kids.items():
            toks[cs] = rng.permutation(V)[:len(cs)]
        lg = rng.standard_normal((1, n, V)).astype(np.float32)
        am = lg[0].argmax(-1)
        best = [0]
        for i in range(n):
            path = []
            u = i
            while u >= 0:
                path.append(u)
                u = int(parent[u])
            path = path[::-1]
            if all(toks[path[j + 1]] == am[path[j]] for j in range(len(path) - 1)) and len(path) > len(best):
                best = path
        an, at, na = oracle.verify_greedy(lg, toks[None], parent[None], [n])
        assert an[0, :na[0]].tolist() == best
        assert at[0, :na[0]].tolist() == [int(toks[c]) for c in best[1:]] + [int(am[best[-1]])]


def test_greedy_tie_rules():
    """Reading R7: argmax ties go to the lowest token id; among children carrying the same
    matching token the lowest node index wins."""
    V = 8
    lg = np.zeros((1, 4, V), np.float32)
    lg[0, 0, [2, 5]] = 3.0          # tie at the root between tokens 2 and 5 -> O(root) = 2
    parent = np.array([[-1, 0, 0, 0]], np.int32)
    toks = np.array([[0, 5, 2, 2]], np.int32)   # nodes 2 and 3 both carry token 2
    an, at, na = oracle.verify_greedy(lg, toks, parent, [4])
    assert an[0, :na[0]].tolist() == [0, 2]
    assert at[0, :na[0]].tolist() == [2, 0]     # then argmax of all-zero logits row = token 0


def test_greedy_invalid_tree():
    lg = np.zeros((1, 3, 4), np.float32)
    an, at, na = oracle.verify_greedy(lg, np.zeros((1, 3), np.int32), np.array([[-1, 2, 0]]), [3])
    assert na[0] == 0 and np.all(an == -1) and np.all(at == -1)


def test_expansion_tree_fig3(golden):
    """Fig. 3 (L476-483, L528): <2,2,1> expands into 11 nodes and 4 sequences."""
    g = golden("fig3_expansion.json")
    parent, depth = W.expansion_tree(g["expansion"])
    assert len(parent) == g["n_nodes"]
    assert parent.tolist() == g["dfs_parent"]
    assert len(set(range(len(parent))) - set(parent.tolist())) == g["n_leaves"]
    # the paper's evaluation config <1,1,3,1,1,1,1,1> (L956-959) has 21 nodes, 3 leaves
    p2, d2 = W.expansion_tree((1, 1, 3, 1, 1, 1, 1, 1))
    assert len(p2) == 21 and d2.max() == 8
