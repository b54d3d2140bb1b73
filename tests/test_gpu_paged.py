"""GPU tests of the NEXT-4 paged KV cache: tree attention and KV commit through a page table
(pages of 128 slots x every kv-head, random page placement) give bit-identical results to the
contiguous calls on the same data, and stay within the attention tolerance of the oracle."""
import numpy as np
import pytest
import torch

import oracle
import workloads as W
from tests.test_gpu_parity import DEV, _check_rows, _oracle_attention, _shape

pytestmark = pytest.mark.gpu

if torch.cuda.is_available():
    import paper_conf_asplos_miaoozcwzwzyssc24_b200 as spi


def _paginate(cache, smax, rng, extra=5):
    """[L][B][Hkv][Smax][128] -> pages [L][num_pages][Hkv][128][128] + page table [B][max_pages]."""
    L, B, H = cache.shape[:3]
    mp = (smax + 127) // 128
    npg = B * mp + extra
    perm = rng.permutation(npg)[:B * mp].reshape(B, mp)
    pages = torch.zeros((L, npg, H, 128, 128), dtype=cache.dtype, device=cache.device)
    for b in range(B):
        for t in range(mp):
            rows = cache[:, b, :, 128 * t:min(128 * (t + 1), smax)]
            pages[:, int(perm[b, t]), :, :rows.shape[2]] = rows
    return pages, torch.from_numpy(perm.astype(np.int32)).to(cache.device)


def _unpaginate(pages, table, smax):
    L, _, H = pages.shape[:3]
    B, mp = table.shape
    out = torch.empty((L, B, H, mp * 128, 128), dtype=pages.dtype, device=pages.device)
    for b in range(B):
        for t in range(mp):
            out[:, b, :, 128 * t:128 * (t + 1)] = pages[:, int(table[b, t])]
    return out[:, :, :, :smax]


@pytest.mark.parametrize("Hq,Hkv,Nmax,P", [(4, 4, 21, 300), (16, 2, 40, 129), (2, 2, 200, 0), (32, 32, 16, 1000)])
def test_paged_attention_bit_identical(Hq, Hkv, Nmax, P):
    rng = np.random.default_rng(P + Nmax)
    B = 3
    trees = [W.random_tree(int(rng.integers(1, Nmax + 1)), 8, 4, rng) for _ in range(B)]
    pls = [P, max(P - 5, 0), P + 77]
    tb = W.make_tree_batch(trees, pls, max_nodes=Nmax, max_depth=8, device=DEV)
    smax = max(pls) + Nmax + 3
    ai = W.make_attention_inputs(tb, 1, Hq, Hkv, smax, seed=P + 3, device=DEV)
    shape = _shape(tb, Hq, Hkv, smax)
    st = spi.TreeState.create(shape, tb.parent, tb.depth, tb.prefix_len, tb.n_nodes)
    st.prepare()
    out_c = torch.full(ai.q.shape[1:], float("nan"), dtype=torch.bfloat16, device=DEV)
    st.attention(ai.q[0], ai.k_cache[0], ai.v_cache[0], out_c)
    kp, table = _paginate(ai.k_cache, smax, rng)
    vp = torch.zeros_like(kp)
    for b in range(B):
        for t in range(table.shape[1]):
            vp[:, int(table[b, t]), :, :min(128, smax - 128 * t)] = ai.v_cache[:, b, :, 128 * t:min(128 * (t + 1), smax)]
    out_p = torch.full_like(out_c, float("nan"))
    spi.specinfer_tree_attention_paged(shape, ai.q[0], kp[0], vp[0], table, tb.parent, tb.depth, tb.prefix_len,
                                       tb.n_nodes, out_p, st.workspace)
    torch.cuda.synchronize()
    n = tb.n_nodes.cpu().numpy()
    for b in range(B):
        assert torch.equal(out_p[b, :n[b]], out_c[b, :n[b]])
    _check_rows(out_p, _oracle_attention(ai, tb), tb)


def test_paged_commit_matches_contiguous():
    rng = np.random.default_rng(11)
    B, L, Hkv = 5, 2, 4
    trees = [W.random_tree(int(rng.integers(2, 30)), 8, 3, rng) for _ in range(B)]
    pls = [int(x) for x in rng.integers(100, 300, B)]   # tree slots straddle page boundaries
    tb = W.make_tree_batch(trees, pls, max_depth=8, device=DEV)
    smax = max(pls) + tb.max_nodes + 2
    ai = W.make_attention_inputs(tb, L, 4, Hkv, smax, seed=7, device=DEV)
    shape = spi.make_shape(B, tb.max_nodes, 4, Hkv, smax, num_layers=L, vocab=64, max_depth=8)
    st = spi.TreeState.create(shape, tb.parent, tb.depth, tb.prefix_len, tb.n_nodes)
    st.prepare()
    vi = W.make_verify_inputs(tb, 64, seed=2, mode="greedy", device=DEV)
    Lp = 9
    an = torch.empty((B, Lp), dtype=torch.int32, device=DEV)
    at, na = torch.empty_like(an), torch.empty((B,), dtype=torch.int32, device=DEV)
    spi.specinfer_verify_greedy(shape, vi.logits, vi.tree_tokens, tb.parent, tb.n_nodes, an, at, na, st.workspace)
    kp, table = _paginate(ai.k_cache, smax, rng)
    # V through the same page table as K
    vp = torch.zeros_like(kp)
    for b in range(B):
        for t in range(table.shape[1]):
            vp[:, int(table[b, t]), :, :min(128, smax - 128 * t)] = ai.v_cache[:, b, :, 128 * t:min(128 * (t + 1), smax)]
    pl_c = tb.prefix_len.clone()
    pl_p = tb.prefix_len.clone()
    k_c, v_c = ai.k_cache.clone(), ai.v_cache.clone()
    spi.specinfer_kv_commit(shape, k_c, v_c, pl_c, an, na)
    spi.specinfer_kv_commit_paged(shape, kp, vp, table, pl_p, an, na)
    torch.cuda.synchronize()
    assert torch.equal(pl_c, pl_p)
    kb, vb = _unpaginate(kp, table, smax), _unpaginate(vp, table, smax)
    for b in range(B):
        P = int(pl_c[b])
        assert torch.equal(kb[:, b, :, :P], k_c[:, b, :, :P]) and torch.equal(vb[:, b, :, :P], v_c[:, b, :, :P])
