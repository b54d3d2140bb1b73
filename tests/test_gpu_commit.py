"""GPU parity of the depth-first KV-cache commit at the
sizes the bench runs, through the C ABI:

  * C2 at full size (32 layers x 16 requests x 32 kv-heads x Smax 2069, 17 GB of cache) and C4 on
    three layers at full batch / heads / prefix / tree, with the accepted paths the GPU verifiers
    produce;
  * the paged commit (NEXT-4) against the oracle through the page table;
  * the bench's kv-head-sharded layout at N = 1 (pack -> gather buffer -> unpack -> commit).

c2's definition: slots [0, P_b) unchanged, slot P_b + j <- old slot P_b + path_b[j] for
j < n_b, P_b += n_b; bit-exact over every slot below the new P_b.  At full size the unchanged prefix
is checked on the device (torch.equal against a copy) and the tree region [P_b, P_b + N) of every
(layer, request, kv-head) goes through the oracle's kv_commit on the host (with prefix 0: c2 only
moves slots relative to P_b).
"""
import numpy as np
import pytest
import torch

import oracle
import workloads as W
from paper_conf_asplos_miaoozcwzwzyssc24_b200 import dist as D
from tests.test_gpu_paged import _paginate, _unpaginate
from tests.test_gpu_parity import DEV

pytestmark = pytest.mark.gpu

if torch.cuda.is_available():
    import paper_conf_asplos_miaoozcwzwzyssc24_b200 as spi


def _bits(t):
    return t.contiguous().cpu().view(torch.int16).numpy().view(np.uint16)


def _check_commit(k0, v0, k1, v1, P0, P1, an, na, N):
    """k0/v0 = cache before, k1/v1 after ([L][B][H][Smax][128], device); P0 / P1 = prefix before /
    after (device); an / na = the accepted paths the commit was given."""
    P0h, P1h = P0.cpu().numpy(), P1.cpu().numpy()
    an_h, na_h = an.cpu().numpy(), na.cpu().numpy()
    np.testing.assert_array_equal(P1h, P0h + np.maximum(na_h, 0))
    B = P0h.shape[0]
    for b in range(B):
        P = int(P0h[b])
        # unchanged committed prefix (on the device)
        assert torch.equal(k1[:, b, :, :P], k0[:, b, :, :P]) and torch.equal(v1[:, b, :, :P], v0[:, b, :, :P])
    # the tree region through the oracle (prefix 0 inside the extracted window)
    for name, c0, c1 in (("K", k0, k1), ("V", v0, v1)):
        win0 = np.stack([_bits(c0[:, b, :, int(P0h[b]):int(P0h[b]) + N]) for b in range(B)], axis=1)
        win1 = np.stack([_bits(c1[:, b, :, int(P0h[b]):int(P0h[b]) + N]) for b in range(B)], axis=1)
        ref_k = np.ascontiguousarray(win0)
        ref_v = np.ascontiguousarray(win0.copy())
        pl = np.zeros(B, np.int32)
        oracle.kv_commit(ref_k, ref_v, pl, an_h, na_h)
        np.testing.assert_array_equal(pl, np.maximum(na_h, 0))
        for b in range(B):
            n = int(pl[b])
            assert np.array_equal(win1[:, b, :, :n], ref_k[:, b, :, :n]), f"{name} request {b}"


def _verify_paths(tb, V, mode, seed, Lp):
    B = tb.parent.shape[0]
    shape = spi.make_shape(B, tb.max_nodes, 1, 1, int(tb.prefix_len.max()) + tb.max_nodes, vocab=V,
                           max_depth=tb.max_depth)
    st = spi.TreeState.create(shape, tb.parent, tb.depth, tb.prefix_len, tb.n_nodes)
    st.prepare()
    vi = W.make_verify_inputs(tb, V, seed=seed, mode=mode, device=DEV)
    an = torch.empty((B, Lp), dtype=torch.int32, device=DEV)
    at, na = torch.empty_like(an), torch.empty((B,), dtype=torch.int32, device=DEV)
    if mode == "greedy":
        spi.specinfer_verify_greedy(shape, vi.logits, vi.tree_tokens, tb.parent, tb.n_nodes, an, at, na,
                                    st.workspace)
    else:
        spi.specinfer_verify_mss(shape, vi.logits, vi.tree_tokens, tb.parent, tb.n_nodes, vi.draft_probs, 1.0,
                                 seed, 0, None, an, at, na, st.workspace)
    torch.cuda.synchronize()
    return an, na


@pytest.mark.parametrize("cfg_name,layers,mode", [("C2", None, "mss"), ("C4", 3, "mss")])
def test_kv_commit_full_size(cfg_name, layers, mode):
    cfg = W.CONFIGS[cfg_name]
    L = layers or cfg.layers
    tb = W.config_tree_batch(cfg, device=DEV)
    B, N = tb.parent.shape
    smax = cfg.prefix + N
    Lp = cfg.max_depth + 1
    an, na = _verify_paths(tb, 4096, mode, cfg.seed, Lp)
    assert int(na.max()) >= 3, "the synthetic drafts should accept a multi-node path somewhere"
    ai = W.make_attention_inputs(tb, 1, cfg.num_kv_heads, cfg.num_kv_heads, smax, seed=cfg.seed, device=DEV,
                                 cache_layers=L)
    k0, v0 = ai.k_cache, ai.v_cache
    k1, v1 = k0.clone(), v0.clone()
    shape = spi.make_shape(B, N, cfg.num_kv_heads, cfg.num_kv_heads, smax, num_layers=L, vocab=4096,
                           max_depth=cfg.max_depth)
    P1 = tb.prefix_len.clone()
    spi.specinfer_kv_commit(shape, k1, v1, P1, an, na)
    torch.cuda.synchronize()
    _check_commit(k0, v0, k1, v1, tb.prefix_len, P1, an, na, N)


def test_paged_commit_against_oracle():
    """The paged commit (NEXT-4) reproduces c2 through the page table: unpaginate, compare with the
    oracle's commit of the contiguous cache (tree slots straddle page boundaries)."""
    rng = np.random.default_rng(21)
    B, L, Hkv = 6, 3, 4
    trees = [W.random_tree(int(rng.integers(2, 40)), 8, 3, rng) for _ in range(B)]
    pls = [int(x) for x in rng.integers(90, 400, B)]
    tb = W.make_tree_batch(trees, pls, max_depth=8, device=DEV)
    smax = max(pls) + tb.max_nodes + 2
    ai = W.make_attention_inputs(tb, L, Hkv, Hkv, smax, seed=12, device=DEV)
    shape = spi.make_shape(B, tb.max_nodes, Hkv, Hkv, smax, num_layers=L, vocab=64, max_depth=8)
    an, na = _verify_paths(tb, 64, "greedy", 3, 9)
    kp, table = _paginate(ai.k_cache, smax, rng)
    # V through the same page table as K
    vp = torch.zeros_like(kp)
    for b in range(B):
        for t in range(table.shape[1]):
            vp[:, int(table[b, t]), :, :min(128, smax - 128 * t)] = ai.v_cache[:, b, :, 128 * t:min(128 * (t + 1), smax)]
    P1 = tb.prefix_len.clone()
    spi.specinfer_kv_commit_paged(shape, kp, vp, table, P1, an, na)
    torch.cuda.synchronize()
    kh, vh = _bits(ai.k_cache).copy(), _bits(ai.v_cache).copy()
    pl = tb.prefix_len.cpu().numpy().copy()
    oracle.kv_commit(kh, vh, pl, an.cpu().numpy(), na.cpu().numpy())
    np.testing.assert_array_equal(pl, P1.cpu().numpy())
    kg, vg = _bits(_unpaginate(kp, table, smax)), _bits(_unpaginate(vp, table, smax))
    for b in range(B):
        e = int(pl[b])
        assert np.array_equal(kg[:, b, :, :e], kh[:, b, :, :e]) and np.array_equal(vg[:, b, :, :e], vh[:, b, :, :e])


def test_kv_shard_layout_n1_commit():
    """bench.py's kv-head-sharded layout at N = 1: the verifier's rows are packed into the gather
    buffer ([n | tokens | nodes], dist.pack_accepted), 'gathered' (a copy at N = 1), unpacked and
    committed into the head shard; the committed cache equals the oracle's commit."""
    cfg = W.CONFIGS["C3"]
    B, P = 4, 300
    tb = W.config_tree_batch(cfg, device=DEV, batch=B)
    tb.prefix_len.fill_(P)
    N = tb.max_nodes
    smax = P + N
    Lp = cfg.max_depth + 1
    an, na = _verify_paths(tb, 2048, "greedy", 5, Lp)
    at = torch.zeros_like(an)
    packed = D.pack_accepted(na, at, an)
    gathered = torch.empty_like(packed)
    gathered.copy_(packed)
    n_all, _, nodes_all = D.unpack_accepted(gathered)
    an_all, na_all = nodes_all.contiguous(), n_all.contiguous()
    kv0, nkv, _, _ = D.shard_kv_heads(cfg.num_q_heads, cfg.num_kv_heads, 2, 1)   # rank 1's shard of 2
    ai = W.make_attention_inputs(tb, 1, cfg.num_kv_heads, cfg.num_kv_heads, smax, seed=7, device=DEV, cache_layers=2)
    k = ai.k_cache[:, :, kv0:kv0 + nkv].contiguous()
    v = ai.v_cache[:, :, kv0:kv0 + nkv].contiguous()
    shape = spi.make_shape(B, N, nkv, nkv, smax, num_layers=2, vocab=2048, max_depth=cfg.max_depth)
    k1, v1, P1 = k.clone(), v.clone(), tb.prefix_len.clone()
    spi.specinfer_kv_commit(shape, k1, v1, P1, an_all, na_all)
    torch.cuda.synchronize()
    _check_commit(k, v, k1, v1, tb.prefix_len, P1, an, na, N)


@pytest.mark.parametrize("join_early", [True, False])
def test_verify_step_concurrent_verifiers_eager_and_graph(join_early):
    """step.VerifyStep with both verifiers (C2's "greedy + MSS"): the MSS verifier runs on a side stream
    concurrently with the committed greedy verifier.  Eager and inside a captured CUDA graph (as bench.py
    replays it), every verifier's outputs equal the plain sequential C-ABI calls, and the committed cache
    equals a commit of the greedy paths."""
    from paper_conf_asplos_miaoozcwzwzyssc24_b200 import step as S
    B, N, Hq, Hkv, P, V, L = 5, 21, 4, 4, 300, 3000, 2
    p_, d_ = W.expansion_tree((1, 1, 3, 1, 1, 1, 1, 1))
    tb = W.make_tree_batch([(p_, d_)] * B, list(W.ragged_prefix(P, B)), device=DEV, max_depth=8)
    Lp = tb.max_depth + 1
    smax = P + N + 3
    ai = W.make_attention_inputs(tb, L, Hq, Hkv, smax, seed=21, device=DEV)
    vi = {m: W.make_verify_inputs(tb, V, seed=22, mode=m, device=DEV) for m in ("greedy", "mss")}
    layout = S.make_layout(B, 1, 0, Hq, Hkv, False)
    shape = spi.make_shape(B, N, Hq, Hkv, smax, num_layers=L, vocab=V, max_depth=tb.max_depth)
    tree = (tb.parent, tb.depth, tb.prefix_len, tb.n_nodes)
    inputs = {m: (vi[m].logits, vi[m].tree_tokens, vi[m].draft_probs if m == "mss" else None) for m in vi}
    rids = torch.arange(B, dtype=torch.int32, device=DEV)

    # reference: the plain calls, one after the other
    st = spi.TreeState.create(shape, *tree)
    st.prepare()
    ref = {}
    for m in ("greedy", "mss"):
        an = torch.empty((B, Lp), dtype=torch.int32, device=DEV)
        at, na = torch.empty_like(an), torch.empty((B,), dtype=torch.int32, device=DEV)
        if m == "greedy":
            spi.specinfer_verify_greedy(shape, vi[m].logits, vi[m].tree_tokens, tb.parent, tb.n_nodes, an, at, na,
                                        st.workspace)
        else:
            spi.specinfer_verify_mss(shape, vi[m].logits, vi[m].tree_tokens, tb.parent, tb.n_nodes, vi[m].draft_probs,
                                     1.0, 7, 0, rids, an, at, na, st.workspace)
        ref[m] = (na.clone(), at.clone(), an.clone())
    k_ref, v_ref, p_ref = ai.k_cache.clone(), ai.v_cache.clone(), tb.prefix_len.clone()
    spi.specinfer_kv_commit(shape, k_ref, v_ref, p_ref, ref["greedy"][2], ref["greedy"][0])
    torch.cuda.synchronize()

    p0 = tb.prefix_len.clone()
    step = S.VerifyStep(S.DeviceOps(), layout, shape, shape, tree, tree, ("greedy", "mss"), Lp, DEV)
    out = torch.empty_like(ai.q)
    k, v = ai.k_cache.clone(), ai.v_cache.clone()

    def one_step():
        tb.prefix_len.copy_(p0)
        step.prepare()
        for l in range(L):
            step.attention(ai.q[l], k[l], v[l], out[l], layer=l)
        step.verify(inputs, seed=7, offset=0, join=join_early)
        step.commit(k, v)     # (join_early False: the commit overlaps the side-stream MSS, as bench.py runs it)
        step.join()

    def check():
        torch.cuda.synchronize()
        for m in ("greedy", "mss"):
            na, at, an = step.accepted(m)
            for x, y in zip((na, at, an), ref[m]):
                assert torch.equal(x, y), m
        assert torch.equal(k, k_ref) and torch.equal(v, v_ref) and torch.equal(tb.prefix_len, p_ref)

    s = torch.cuda.Stream()
    s.wait_stream(torch.cuda.current_stream())
    with torch.cuda.stream(s):
        one_step()
    check()
    g = torch.cuda.CUDAGraph()
    k.copy_(ai.k_cache), v.copy_(ai.v_cache)
    with torch.cuda.graph(g, stream=s):
        one_step()
    for _ in range(2):
        k.copy_(ai.k_cache), v.copy_(ai.v_cache)
        for m in ("greedy", "mss"):
            for t_ in step.res[m]:
                t_.fill_(-5)
        torch.cuda.synchronize()
        g.replay()
        check()
