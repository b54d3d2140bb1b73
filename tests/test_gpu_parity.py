"""GPU parity: the CUDA path (through the C ABI) against the fp64 CPU oracle.

Bars (BASELINE.json north_star): tree attention max|err| <= 1e-2 and mean|err| <= 1e-3 on the
same bf16-rounded inputs; greedy verification, KV commit and accepted paths bit-exact; MSS
bit-exact except decisions whose relative margin is < 1e-5 (fp32 vs fp64).
"""
import numpy as np
import pytest
import torch

import oracle
import workloads as W
from tests.mss_compare import compare_sampled

pytestmark = pytest.mark.gpu

if torch.cuda.is_available():
    import paper_conf_asplos_miaoozcwzwzyssc24_b200 as spi

MAX_ABS, MEAN_ABS = 1e-2, 1e-3
DEV = "cuda:0"


def _shape(tb, Hq, Hkv, smax, **kw):
    return spi.make_shape(tb.parent.shape[0], tb.max_nodes, Hq, Hkv, smax, max_depth=tb.max_depth, **kw)


def _gpu_attention(tb, ai, Hq, Hkv, layer=0, sm_scale=0.0):
    shape = _shape(tb, Hq, Hkv, ai.smax, sm_scale=sm_scale)
    st = spi.TreeState.create(shape, tb.parent, tb.depth, tb.prefix_len, tb.n_nodes)
    st.prepare()
    out = torch.full(ai.q.shape[1:], float("nan"), dtype=torch.bfloat16, device=DEV)
    st.attention(ai.q[layer], ai.k_cache[layer], ai.v_cache[layer], out)
    torch.cuda.synchronize()
    return out, st


def _check_rows(got, ref, tb, bs=None, heads=None):
    n = tb.n_nodes.cpu().numpy()
    bs = range(got.shape[0]) if bs is None else bs
    errs = []
    for b in bs:
        g = got[b, :n[b]].float().cpu().numpy()
        r = ref[b, :n[b]]
        if heads is not None:
            g, r = g[:, heads], r[:, heads]
        assert np.all(np.isfinite(g)), f"non-finite output in request {b}"
        errs.append(np.abs(g - r).reshape(-1))
    e = np.concatenate(errs)
    assert e.max() <= MAX_ABS and e.mean() <= MEAN_ABS, (e.max(), e.mean())
    return e.max(), e.mean()


def _oracle_attention(ai, tb, layer=0, bs=None):
    q, k, v = ai.q[layer].cpu(), ai.k_cache[layer].cpu(), ai.v_cache[layer].cpu()
    par, dep, pl, nn_ = tb.parent.cpu(), tb.depth.cpu(), tb.prefix_len.cpu(), tb.n_nodes.cpu()
    if bs is None:
        return oracle.tree_attention(q, k, v, par, dep, pl, nn_)
    ref = np.full(q.shape, np.nan)
    for b in bs:
        ref[b:b + 1] = oracle.tree_attention(q[b:b + 1], k[b:b + 1], v[b:b + 1], par[b:b + 1], dep[b:b + 1],
                                             pl[b:b + 1], nn_[b:b + 1])
    return ref


# ---------------------------------------------------------------------------------------------
# tree attention
# ---------------------------------------------------------------------------------------------

@pytest.mark.parametrize("Hq,Hkv,Nmax", [(2, 2, 8), (8, 4, 4), (4, 4, 16), (4, 2, 16), (2, 2, 32),
                                         (8, 1, 8), (4, 4, 64), (8, 2, 20), (3, 3, 100), (16, 2, 40),
                                         (1, 1, 256)])
@pytest.mark.parametrize("P", [0, 1, 127, 128, 300])
def test_attention_random_trees(Hq, Hkv, Nmax, P):
    """Random trees (ragged n_b), ragged prefixes around tile boundaries, NaN-poisoned unused
    cache slots; covers NT = 16/32/64 and multi-chunk items."""
    B = 3
    rng = np.random.default_rng(1000 * Hq + 10 * Nmax + P)
    trees = [W.random_tree(int(rng.integers(1, Nmax + 1)), 8, 4, rng) for _ in range(B)]
    pls = [P, max(P - 1, 0), P + 45]
    tb = W.make_tree_batch(trees, pls, max_nodes=Nmax, max_depth=8, device=DEV)
    smax = max(pls) + Nmax + 7
    ai = W.make_attention_inputs(tb, 1, Hq, Hkv, smax, seed=P + Nmax, device=DEV, poison=True)
    out, _ = _gpu_attention(tb, ai, Hq, Hkv)
    ref = _oracle_attention(ai, tb)
    _check_rows(out, ref, tb)
    # padded rows are untouched
    n = tb.n_nodes.cpu().numpy()
    for b in range(B):
        assert torch.isnan(out[b, n[b]:].float()).all()


@pytest.mark.parametrize("Hq,Hkv,Nmax", [(4, 4, 16), (2, 2, 100), (8, 1, 40)])
@pytest.mark.parametrize("spike", [8.0, 30.0, 200.0])
def test_attention_score_spikes(Hq, Hkv, Nmax, spike):
    """Keys scaled by large factors inside later chunks / tiles (committed and tree keys), so a row's
    running softmax reference has to move mid-tile and across tiles by far more than any stale-max
    slack; with spike 200 the scores jump by hundreds of log2 units (one-hot rows)."""
    B = 2
    rng = np.random.default_rng(int(spike) + Nmax)
    trees = [W.random_tree(Nmax, 8, 4, rng), W.random_tree(int(rng.integers(1, Nmax + 1)), 8, 4, rng)]
    P = 300
    pls = [P, P - 100]
    tb = W.make_tree_batch(trees, pls, max_nodes=Nmax, max_depth=8, device=DEV)
    smax = max(pls) + Nmax + 7
    ai = W.make_attention_inputs(tb, 1, Hq, Hkv, smax, seed=int(spike), device=DEV, poison=True)
    for b, pb in enumerate(pls):
        for j, f in ((70, spike / 4), (150, spike / 2), (pb - 1, spike), (pb + 3, spike * 1.5)):
            ai.k_cache[0, b, :, j] = (ai.k_cache[0, b, :, j].float() * f).to(torch.bfloat16)
    out, _ = _gpu_attention(tb, ai, Hq, Hkv)
    ref = _oracle_attention(ai, tb)
    # near one-hot rows: |out| reaches |v| ~ 4, where one bf16 rounding of the output alone is up
    # to 2^-7 = 0.0078; the 1e-2 absolute bar assumes |out| <~ 1, so it is
    # applied relative to max(1, |ref|) here
    n = tb.n_nodes.cpu().numpy()
    for b in range(B):
        g = out[b, :n[b]].float().cpu().numpy()
        r = ref[b, :n[b]]
        e = np.abs(g - r)
        assert np.all(e <= MAX_ABS * np.maximum(1.0, np.abs(r))) and e.mean() <= MEAN_ABS, (b, e.max(), e.mean())


@pytest.mark.parametrize("Hq,Hkv,pls", [(4, 4, [3000]), (8, 2, [3000, 100]), (16, 8, [1700, 2900, 40])])
def test_attention_split_kv_clusters(Hq, Hkv, pls):
    """Split-KV mode (few items: each item's tiles split over a thread-block cluster of up to 8 CTAs,
    merged through DSMEM by rank 0; items shorter than 12 tiles stay whole on rank 0), ragged prefixes
    and trees, NaN-poisoned unused cache slots."""
    rng = np.random.default_rng(sum(pls) + Hq)
    Nmax = 24
    B = len(pls)
    trees = [W.random_tree(int(rng.integers(1, Nmax + 1)), 8, 4, rng) for _ in range(B)]
    tb = W.make_tree_batch(trees, pls, max_nodes=Nmax, max_depth=8, device=DEV)
    smax = max(pls) + Nmax + 5
    ai = W.make_attention_inputs(tb, 1, Hq, Hkv, smax, seed=len(pls) + Hq, device=DEV, poison=True)
    out, _ = _gpu_attention(tb, ai, Hq, Hkv)
    ref = _oracle_attention(ai, tb)
    _check_rows(out, ref, tb)
    n = tb.n_nodes.cpu().numpy()
    for b in range(B):
        assert torch.isnan(out[b, n[b]:].float()).all()


@pytest.mark.parametrize("case", ["staged", "batched"])
def test_attention_split_merge_paths(case):
    """Stream-K split items (units cut by CTA boundaries) and both merge paths of the last piece:
    'staged' = every piece's (O, m, l) bulk-copied into the idle K/V rings (at most 8 pieces);
    'batched' = one request whose KV stream spans far more than 8 CTAs' shares, so its merge runs
    the batched-load path (pieces read 8 at a time)."""
    if case == "staged":
        # 24 units x ~24 tiles over 148 CTAs: stream-K (a unit exceeds an even share by > 8 tiles),
        # every unit cut into ~6 pieces
        B, Hq, Hkv, P = 3, 8, 8, 3000
        parent, depth = W.expansion_tree((1, 1, 3, 1, 1, 1, 1, 1))
        pls = list(W.ragged_prefix(P, B))
        trees = [(parent, depth)] * B
    else:
        # 40 single-head requests, one of them with a 40000-key prefix (~313 tiles = ~130 CTAs'
        # shares of the ~350-tile stream): that item is cut into far more than 8 pieces
        B, Hq, Hkv = 40, 2, 1
        parent, depth = W.expansion_tree((1, 2, 2))
        pls = [40000] + [5 + 3 * b for b in range(B - 1)]
        trees = [(parent, depth)] * B
    tb = W.make_tree_batch(trees, pls, device=DEV, max_depth=8)
    smax = max(pls) + tb.max_nodes + 3
    ai = W.make_attention_inputs(tb, 1, Hq, Hkv, smax, seed=77, device=DEV, poison=True)
    out, _ = _gpu_attention(tb, ai, Hq, Hkv)
    ref = _oracle_attention(ai, tb)
    _check_rows(out, ref, tb)


@pytest.mark.parametrize("peaky", [False, True])
def test_attention_chain_and_figures(golden, peaky):
    """Fig. 4 tree (L682), a 40-node chain (= causal decoding), root-only trees; peaky q (x4)
    stresses the online-softmax rescaling."""
    g = golden("fig4_mask.json")
    fig4 = (np.asarray(g["parent"], np.int32), None)
    p4 = fig4[0]
    d4 = np.zeros(len(p4), np.int32)
    for i in range(1, len(p4)):
        d4[i] = d4[p4[i]] + 1
    trees = [(p4, d4), W.chain_tree(40), (np.array([-1], np.int32), np.array([0], np.int32)),
             W.expansion_tree((2, 2, 1))]
    tb = W.make_tree_batch(trees, [0, 513, 700, 5], max_nodes=40, max_depth=39, device=DEV)
    smax = 800
    ai = W.make_attention_inputs(tb, 1, 8, 8, smax, seed=7, device=DEV, peaky=peaky, poison=True)
    out, _ = _gpu_attention(tb, ai, 8, 8)
    _check_rows(out, _oracle_attention(ai, tb), tb)


def test_attention_custom_scale_and_empty_prefix():
    trees = [W.expansion_tree((3, 3))] * 2
    tb = W.make_tree_batch(trees, [0, 0], device=DEV)
    ai = W.make_attention_inputs(tb, 1, 4, 4, 20, seed=3, device=DEV, poison=True)
    out, _ = _gpu_attention(tb, ai, 4, 4, sm_scale=0.2)
    ref = oracle.tree_attention(ai.q[0].cpu(), ai.k_cache[0].cpu(), ai.v_cache[0].cpu(), tb.parent.cpu(),
                                tb.depth.cpu(), tb.prefix_len.cpu(), tb.n_nodes.cpu(), sm_scale=0.2)
    _check_rows(out, ref, tb)


def test_attention_invalid_tree_status():
    """A bad tree sets the sticky device status and leaves its rows untouched; other requests
    are computed normally."""
    trees = [W.expansion_tree((2, 2)), W.expansion_tree((2, 2))]
    tb = W.make_tree_batch(trees, [10, 10], device=DEV)
    tb.parent[1, 3] = 5   # parent not < i
    ai = W.make_attention_inputs(tb, 1, 2, 2, 30, seed=4, device=DEV)
    out, st = _gpu_attention(tb, ai, 2, 2)
    assert spi.specinfer_read_device_status(st.workspace) & 1
    assert torch.isnan(out[1].float()).all()
    ref = _oracle_attention(ai, tb)
    _check_rows(out, ref, tb, bs=[0])


@pytest.mark.parametrize("Hq,Hkv,expansion,B", [(32, 32, (1, 1, 3, 1, 1, 1, 1, 1), 24),   # swapped, 768 items
                                                 (64, 8, (1, 2, 2, 2, 2, 2), 8)])            # rows, 256 items
def test_dynamic_schedule_with_invalid_requests(Hq, Hkv, expansion, B):
    """Enough items per CTA for the dynamic whole-item schedule (ticket counter), with two invalid
    trees among the requests: their items are empty (skipped by the claims), their rows stay
    untouched, every other request matches the oracle; a second call on the same workspace (the
    next layer: tickets continue from the first call's) gives bit-identical rows."""
    parent, depth = W.expansion_tree(expansion)
    pls = [300 + 37 * b for b in range(B)]
    tb = W.make_tree_batch([(parent, depth)] * B, pls, device=DEV, max_depth=8)
    tb.parent[3, 2] = 7    # parent not < i
    tb.parent[B - 2, 1] = 1
    ai = W.make_attention_inputs(tb, 2, Hq, Hkv, max(pls) + tb.max_nodes + 1, seed=8, device=DEV)
    out, st = _gpu_attention(tb, ai, Hq, Hkv)
    assert spi.specinfer_read_device_status(st.workspace) & 1
    for bad in (3, B - 2):
        assert torch.isnan(out[bad].float()).all()
    again = torch.full_like(out, float("nan"))
    st.attention(ai.q[0], ai.k_cache[0], ai.v_cache[0], again)
    torch.cuda.synchronize()
    assert torch.equal(torch.nan_to_num(again, nan=7.0), torch.nan_to_num(out, nan=7.0))
    bs = [0, 1, B - 1]
    _check_rows(out, _oracle_attention(ai, tb, bs=bs), tb, bs=bs)


@pytest.mark.parametrize("Br,Bs", [(2, 18), (3, 19)])
def test_schedule_mode_boundaries(Br, Bs):
    """Either side of the schedule switches (148-SM grid): the rows kernel claims whole items from
    n_items >= 74 (half an item per CTA; Br x 8 kv-heads x 4 chunks = 64 / 96 items), the swapped kernel
    from n_items >= 148 (Bs x 8 kv-heads = 144 / 152 items); sampled requests vs the oracle."""
    parent, depth = W.expansion_tree((1, 2, 2, 2, 2, 2))        # 63 nodes: rows kernel at G = 8 (4 chunks)
    tb = W.make_tree_batch([(parent, depth)] * Br, [150 + 11 * b for b in range(Br)], device=DEV, max_depth=8)
    ai = W.make_attention_inputs(tb, 1, 64, 8, 150 + 11 * Br + tb.max_nodes, seed=Br, device=DEV, poison=True)
    out, _ = _gpu_attention(tb, ai, 64, 8)
    _check_rows(out, _oracle_attention(ai, tb), tb)
    parent, depth = W.expansion_tree((1, 1, 3, 1, 1, 1, 1, 1))  # 21 nodes: swapped kernel, 1 chunk
    tb = W.make_tree_batch([(parent, depth)] * Bs, [300 + 7 * b for b in range(Bs)], device=DEV, max_depth=8)
    ai = W.make_attention_inputs(tb, 1, 8, 8, 300 + 7 * Bs + tb.max_nodes, seed=Bs, device=DEV, poison=True)
    out, _ = _gpu_attention(tb, ai, 8, 8)
    bs = [0, Bs // 2, Bs - 1]
    _check_rows(out, _oracle_attention(ai, tb, bs=bs), tb, bs=bs)


def test_rows_kernel_dynamic_ragged_chunks():
    """Rows kernel in the dynamic whole-item mode with two 128-row chunks per (request, kv-head) and
    ragged trees: requests with 15 nodes leave their second chunk empty (skipped by the claims), requests
    with 129 nodes fill both; sampled requests of both kinds match the oracle."""
    big, small = W.expansion_tree((2, 3, 4, 4)), W.expansion_tree((2, 2, 2))
    B = 48
    trees = [big if b % 2 == 0 else small for b in range(B)]
    pls = [200 + 13 * b for b in range(B)]
    tb = W.make_tree_batch(trees, pls, device=DEV, max_depth=8)
    ai = W.make_attention_inputs(tb, 1, 4, 4, max(pls) + tb.max_nodes + 1, seed=12, device=DEV, poison=True)
    out, _ = _gpu_attention(tb, ai, 4, 4)
    bs = [0, 1, B - 2, B - 1]
    _check_rows(out, _oracle_attention(ai, tb, bs=bs), tb, bs=bs)


@pytest.mark.parametrize("name,batch", [("C2", 3), ("C3", 2), ("C1", 1)])
def test_prepare_initialises_a_garbage_workspace(name, batch):
    """tree_prepare needs no zeroed workspace (no memset since round 2): with every byte of the workspace
    set to 0xFF first, prepare -> attention -> greedy verify -> MSS verify -> KV commit give bit-identical
    results to a zero-filled workspace, twice in a row (counters re-armed by the calls themselves); a bad
    tree's status bit is cleared by the next prepare of a good tree."""
    cfg = W.CONFIGS[name]
    tb = W.config_tree_batch(cfg, device=DEV, ragged=True, batch=batch)
    smax = cfg.prefix + tb.max_nodes + 3
    ai = W.make_attention_inputs(tb, 1, cfg.num_q_heads, cfg.num_kv_heads, smax, seed=11, device=DEV)
    V = 4000
    vg = W.make_verify_inputs(tb, V, seed=12, mode="greedy", device=DEV)
    vm = W.make_verify_inputs(tb, V, seed=13, mode="mss", device=DEV)
    shape = spi.make_shape(batch, tb.max_nodes, cfg.num_q_heads, cfg.num_kv_heads, smax, vocab=V,
                           max_depth=tb.max_depth)
    B, Lp = batch, tb.max_depth + 1

    def run(fill):
        ws = spi.alloc_workspace(shape, DEV)
        ws.fill_(fill)
        st = spi.TreeState.create(shape, tb.parent, tb.depth, tb.prefix_len, tb.n_nodes, workspace=ws)
        res = []
        for _ in range(2):
            k, v, pl = ai.k_cache.clone(), ai.v_cache.clone(), tb.prefix_len.clone()
            st.prefix_len = pl
            st.prepare()
            out = torch.full(ai.q.shape[1:], float("nan"), dtype=torch.bfloat16, device=DEV)
            st.attention(ai.q[0], k[0], v[0], out)
            outs = [out]
            for mode, vi in (("greedy", vg), ("mss", vm)):
                an = torch.empty((B, Lp), dtype=torch.int32, device=DEV)
                at, na = torch.empty_like(an), torch.empty((B,), dtype=torch.int32, device=DEV)
                if mode == "greedy":
                    spi.specinfer_verify_greedy(shape, vi.logits, vi.tree_tokens, tb.parent, tb.n_nodes, an, at, na,
                                                ws)
                else:
                    spi.specinfer_verify_mss(shape, vi.logits, vi.tree_tokens, tb.parent, tb.n_nodes, vi.draft_probs,
                                             1.0, 5, 0, None, an, at, na, ws)
                outs += [an, at, na]
            spi.specinfer_kv_commit(shape, k, v, pl, outs[1], outs[3])
            outs += [k, v, pl]
            torch.cuda.synchronize()
            assert spi.specinfer_read_device_status(ws) == 0
            res.append([torch.nan_to_num(x.float(), nan=7.0).cpu() if x.is_floating_point() else x.cpu() for x in outs])
        return ws, st, res

    _, _, r0 = run(0)
    ws, st, r1 = run(255)
    for a_, b_ in ((r0[0], r1[0]), (r0[1], r1[1]), (r0[0], r0[1])):
        for x, y in zip(a_, b_):
            assert torch.equal(x, y)
    # status: a bad tree sets the bit, the next good prepare clears it
    bad = tb.parent.clone()
    bad[0, min(2, int(tb.n_nodes[0]) - 1)] = 99
    st.parent = bad
    st.prepare()
    torch.cuda.synchronize()
    assert spi.specinfer_read_device_status(ws) & 1
    st.parent = tb.parent
    st.prepare()
    torch.cuda.synchronize()
    assert spi.specinfer_read_device_status(ws) == 0


def test_host_validation_errors():
    tb = W.make_tree_batch([W.chain_tree(4)], [3], device=DEV)
    ai = W.make_attention_inputs(tb, 1, 2, 2, 16, seed=5, device=DEV)
    shape = _shape(tb, 2, 2, 16)
    st = spi.TreeState.create(shape, tb.parent, tb.depth, tb.prefix_len, tb.n_nodes)
    out = torch.empty(ai.q.shape[1:], dtype=torch.bfloat16, device=DEV)
    with pytest.raises(ValueError):
        st.attention(ai.q[0].float(), ai.k_cache[0], ai.v_cache[0], out)
    with pytest.raises(ValueError):
        st.attention(ai.q[0], ai.k_cache[0].cpu(), ai.v_cache[0], out)
    bad = spi.make_shape(1, 4, 2, 2, 16, head_dim=64)
    with pytest.raises(spi.SpecInferError):
        spi.specinfer_tree_prepare(bad, tb.parent, tb.depth, tb.prefix_len, tb.n_nodes, st.workspace)


def test_attention_cuda_graph_replay():
    """The calls are stream-ordered and graph-capturable (bench.py replays a CUDA graph)."""
    cfg = W.CONFIGS["C1"]
    tb = W.config_tree_batch(cfg, device=DEV)
    smax = cfg.prefix + tb.max_nodes
    ai = W.make_attention_inputs(tb, 1, 32, 32, smax, seed=1, device=DEV)
    shape = _shape(tb, 32, 32, smax)
    st = spi.TreeState.create(shape, tb.parent, tb.depth, tb.prefix_len, tb.n_nodes)
    out = torch.zeros(ai.q.shape[1:], dtype=torch.bfloat16, device=DEV)
    s = torch.cuda.Stream()
    with torch.cuda.stream(s):
        st.prepare()
        st.attention(ai.q[0], ai.k_cache[0], ai.v_cache[0], out)
    torch.cuda.synchronize()
    first = out.clone()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=s):
        st.prepare()
        st.attention(ai.q[0], ai.k_cache[0], ai.v_cache[0], out)
    out.zero_()
    for _ in range(3):
        g.replay()
    torch.cuda.synchronize()
    assert torch.equal(out, first)


# ---------------------------------------------------------------------------------------------
# the BASELINE.json configs at full size (attention: one layer per config; each layer is an
# independent call of the same kernel in the same launch configuration bench.py times)
# ---------------------------------------------------------------------------------------------

def test_config_c1_full():
    cfg = W.CONFIGS["C1"]
    tb = W.config_tree_batch(cfg, device=DEV)
    smax = cfg.prefix + tb.max_nodes
    ai = W.make_attention_inputs(tb, 1, cfg.num_q_heads, cfg.num_kv_heads, smax, seed=cfg.seed, device=DEV)
    out, _ = _gpu_attention(tb, ai, cfg.num_q_heads, cfg.num_kv_heads)
    _check_rows(out, _oracle_attention(ai, tb), tb)


@pytest.mark.parametrize("name,bs,heads", [("C2", [0, 7, 15], None), ("C3", [0, 31], list(range(8, 16))),
                                           ("C4", [0, 63], [0, 1, 55])])
def test_config_full_size_sampled(name, bs, heads):
    """Full batch/prefix/tree of the config (ragged prefixes), one layer; sampled requests and
    heads against the oracle, every row against an fp32 torch reference on the GPU."""
    cfg = W.CONFIGS[name]
    tb = W.config_tree_batch(cfg, device=DEV, ragged=True)
    smax = cfg.prefix + tb.max_nodes + 3
    ai = W.make_attention_inputs(tb, 1, cfg.num_q_heads, cfg.num_kv_heads, smax, seed=cfg.seed, device=DEV,
                                 poison=True)
    out, _ = _gpu_attention(tb, ai, cfg.num_q_heads, cfg.num_kv_heads)
    if heads is not None:
        q = ai.q[0][:, :, heads].contiguous()
        G = cfg.num_q_heads // cfg.num_kv_heads
        kvh = sorted({h // G for h in heads})
        # oracle on the sampled requests with only the needed heads: remap heads to a small GQA problem
        ref_full = np.full((len(bs), tb.max_nodes, len(heads), 128), np.nan)
        for bi, b in enumerate(bs):
            for hi, h in enumerate(heads):
                g = h // G
                r = oracle.tree_attention(ai.q[0][b:b + 1, :, h:h + 1].cpu(), ai.k_cache[0][b:b + 1, g:g + 1].cpu(),
                                          ai.v_cache[0][b:b + 1, g:g + 1].cpu(), tb.parent[b:b + 1].cpu(),
                                          tb.depth[b:b + 1].cpu(), tb.prefix_len[b:b + 1].cpu(),
                                          tb.n_nodes[b:b + 1].cpu())
                ref_full[bi, :, hi] = r[0, :, 0]
        n = tb.n_nodes.cpu().numpy()
        for bi, b in enumerate(bs):
            g = out[b, :n[b], heads].float().cpu().numpy()
            e = np.abs(g - ref_full[bi, :n[b]])
            assert e.max() <= MAX_ABS and e.mean() <= MEAN_ABS, (b, e.max(), e.mean())
    else:
        ref = _oracle_attention(ai, tb, bs=bs)
        _check_rows(out, ref, tb, bs=bs)
    # every row: fp32 torch reference on the GPU (secondary check, not the parity oracle)
    _torch_reference_check(out, ai, tb, cfg.num_q_heads, cfg.num_kv_heads)


def _torch_reference_check(out, ai, tb, Hq, Hkv):
    B, N = tb.parent.shape
    G = Hq // Hkv
    anc = torch.zeros((B, N, N), dtype=torch.bool, device=DEV)
    par = tb.parent.cpu().numpy()
    n = tb.n_nodes.cpu().numpy()
    for b in range(B):
        for i in range(n[b]):
            u = i
            while u >= 0:
                anc[b, i, u] = True
                u = par[b, u]
    pl = tb.prefix_len
    for b in range(B):
        P, nb = int(pl[b]), int(n[b])
        k = ai.k_cache[0, b, :, :P + nb].float()
        v = ai.v_cache[0, b, :, :P + nb].float()
        q = ai.q[0, b, :nb].float().permute(1, 0, 2)          # [Hq][nb][D]
        mask = torch.ones((nb, P + nb), dtype=torch.bool, device=DEV)
        mask[:, P:] = anc[b, :nb, :nb]
        ref = torch.nn.functional.scaled_dot_product_attention(
            q, k.repeat_interleave(G, 0), v.repeat_interleave(G, 0), attn_mask=mask)
        e = (out[b, :nb].float().permute(1, 0, 2) - ref).abs()
        assert e.max().item() <= MAX_ABS and e.mean().item() <= MEAN_ABS


@pytest.mark.parametrize("name,batch", [("C4", 16), ("C3", 32), ("C2", 16)])
def test_attention_rescales_across_segments(name, batch):
    """Production shapes (every CTA runs many segments) with keys ramped along the sequence, so the
    rows' running reference moves on most tiles (stale-max rescales of O) while the softmax groups
    hand decisions and segment ends to each other.  Eight launches must be bit-identical (the two
    latent races this guards against -- a shared decision barrier that the publisher could complete
    itself, and an ambiguous parity wait before a rescale -- made the rows kernel non-deterministic
    here), and every row must match an fp32 torch reference, sampled rows the oracle."""
    cfg = W.CONFIGS[name]
    tb = W.config_tree_batch(cfg, device=DEV, ragged=True, batch=batch)
    smax = cfg.prefix + tb.max_nodes + 3
    ai = W.make_attention_inputs(tb, 1, cfg.num_q_heads, cfg.num_kv_heads, smax, seed=cfg.seed + 5, device=DEV)
    ramp = torch.linspace(0.2, 3.0, smax, device=DEV).view(1, 1, smax, 1)
    ai.k_cache[0].copy_((ai.k_cache[0].float() * ramp).to(torch.bfloat16))
    out, st = _gpu_attention(tb, ai, cfg.num_q_heads, cfg.num_kv_heads)
    for _ in range(7):
        again = torch.full_like(out, float("nan"))
        st.attention(ai.q[0], ai.k_cache[0], ai.v_cache[0], again)
        torch.cuda.synchronize()
        assert torch.equal(torch.nan_to_num(again, nan=7.0), torch.nan_to_num(out, nan=7.0))
    # fp32 torch reference, every row; the bar is relative to max(1, |ref|) as in the spike test
    # (peaked rows: |out| approaches |v|, where one bf16 rounding of the output is ~|v| 2^-8)
    B, N = tb.parent.shape
    G = cfg.num_q_heads // cfg.num_kv_heads
    par, n, pl = tb.parent.cpu().numpy(), tb.n_nodes.cpu().numpy(), tb.prefix_len.cpu().numpy()
    for b in range(B):
        P, nb = int(pl[b]), int(n[b])
        mask = torch.ones((nb, P + nb), dtype=torch.bool, device=DEV)
        anc = torch.zeros((nb, nb), dtype=torch.bool)
        for i in range(nb):
            u = i
            while u >= 0:
                anc[i, u] = True
                u = par[b, u]
        mask[:, P:] = anc.to(DEV)
        k = ai.k_cache[0, b, :, :P + nb].float().repeat_interleave(G, 0)
        v = ai.v_cache[0, b, :, :P + nb].float().repeat_interleave(G, 0)
        ref = torch.nn.functional.scaled_dot_product_attention(ai.q[0, b, :nb].float().permute(1, 0, 2), k, v,
                                                               attn_mask=mask)
        e = (out[b, :nb].float().permute(1, 0, 2) - ref).abs()
        assert (e <= MAX_ABS * ref.abs().clamp(min=1.0)).all() and e.mean().item() <= MEAN_ABS, (b, e.max().item())
    ref_o = _oracle_attention(ai, tb, bs=[0])
    g = out[0, :n[0]].float().cpu().numpy()
    e = np.abs(g - ref_o[0, :n[0]])
    assert np.all(e <= MAX_ABS * np.maximum(1.0, np.abs(ref_o[0, :n[0]]))) and e.mean() <= MEAN_ABS


@pytest.mark.parametrize("case", ["five_pieces", "many_pieces"])
def test_rows_kernel_split_merge_paths(case):
    """Rows-as-M kernel (G * Nmax > 64) with stream-K split units, merged by the epilogue warpgroup:
    'five_pieces' = 32 MHA units of 65 tiles over 148 CTAs (each unit cut into ~5 pieces: more than one
    staging round of the idle rings); 'many_pieces' = one 40000-key request among short ones (its unit is
    cut into ~100 pieces: the batched-load merge and the multi-round staged merge)."""
    if case == "five_pieces":
        tb = W.random_tree_batch(1, 128, 8192, seed=11, device=DEV)
        Hq = Hkv = 32
    else:
        parent, depth = W.expansion_tree((2, 3, 4, 4))   # 129 nodes: two 128-row blocks (lock-step lanes)
        B = 6
        pls = [40000] + [5 + 97 * b for b in range(B - 1)]
        tb = W.make_tree_batch([(parent, depth)] * B, pls, device=DEV, max_depth=8)
        Hq = Hkv = 2
    smax = int(tb.prefix_len.max()) + tb.max_nodes + 1
    ai = W.make_attention_inputs(tb, 1, Hq, Hkv, smax, seed=21, device=DEV, poison=True)
    out, _ = _gpu_attention(tb, ai, Hq, Hkv)
    bs = [0] if tb.parent.shape[0] == 1 else [0, tb.parent.shape[0] - 1]
    _check_rows(out, _oracle_attention(ai, tb, bs=bs), tb, bs=bs)


@pytest.mark.parametrize("n,B,P", [(8, 64, 512), (32, 8, 2048), (128, 4, 8192), (256, 2, 2048), (64, 1, 512)])
def test_config_c5_points(n, B, P):
    """C5 sweep points (random trees, depth <= 8), one layer, sampled requests vs the oracle."""
    tb = W.random_tree_batch(B, n, P, seed=n + B + P, device=DEV)
    smax = P + n
    ai = W.make_attention_inputs(tb, 1, 32, 32, smax, seed=5, device=DEV)
    out, _ = _gpu_attention(tb, ai, 32, 32)
    bs = [0, B - 1] if B > 1 else [0]
    _check_rows(out, _oracle_attention(ai, tb, bs=bs), tb, bs=bs)


# ---------------------------------------------------------------------------------------------
# verification
# ---------------------------------------------------------------------------------------------

def _verify_setup(tb, V, mode, seed, Hq=2, Hkv=2):
    smax = int(tb.prefix_len.max()) + tb.max_nodes + 1
    shape = _shape(tb, Hq, Hkv, smax, vocab=V)
    st = spi.TreeState.create(shape, tb.parent, tb.depth, tb.prefix_len, tb.n_nodes)
    st.prepare()
    vi = W.make_verify_inputs(tb, V, seed=seed, mode=mode, device=DEV)
    B, Lp = tb.parent.shape[0], tb.max_depth + 1
    outs = [torch.empty((B, Lp), dtype=torch.int32, device=DEV), torch.empty((B, Lp), dtype=torch.int32, device=DEV),
            torch.empty((B,), dtype=torch.int32, device=DEV)]
    return shape, st, vi, outs


@pytest.mark.parametrize("V", [7, 1000, 32000, 50272])
def test_verify_greedy_parity(V):
    rng = np.random.default_rng(V)
    trees = [W.random_tree(int(rng.integers(1, 60)), 8, 4, rng) for _ in range(12)]
    tb = W.make_tree_batch(trees, [5] * 12, max_nodes=64, max_depth=8, device=DEV)
    shape, st, vi, (an, at, na) = _verify_setup(tb, V, "greedy", seed=V)
    spi.specinfer_verify_greedy(shape, vi.logits, vi.tree_tokens, tb.parent, tb.n_nodes, an, at, na, st.workspace)
    torch.cuda.synchronize()
    r = oracle.verify_greedy(vi.logits.cpu().numpy(), vi.tree_tokens.cpu().numpy(), tb.parent.cpu().numpy(),
                             tb.n_nodes.cpu().numpy(), path_len=9)
    for x, y in zip(r, (an, at, na)):
        assert np.array_equal(x, y.cpu().numpy())
    # repeated call on the same workspace (counters reset) gives the same answer
    spi.specinfer_verify_greedy(shape, vi.logits, vi.tree_tokens, tb.parent, tb.n_nodes, an, at, na, st.workspace)
    torch.cuda.synchronize()
    assert np.array_equal(r[2], na.cpu().numpy())


def test_verify_greedy_fig2_and_ties(golden):
    g = golden("fig2_greedy.json")
    vocab = {w: i for i, w in enumerate(g["vocab"])}
    par = np.asarray(g["parent"], np.int32)
    dep = np.zeros(len(par), np.int32)
    for i in range(1, len(par)):
        dep[i] = dep[par[i]] + 1
    tb = W.make_tree_batch([(par, dep)], [0], max_depth=int(dep.max()), device=DEV)
    shape, st, vi, (an, at, na) = _verify_setup(tb, len(vocab), "greedy", seed=1)
    lg = torch.zeros((1, len(par), len(vocab)), device=DEV)
    for u, w in enumerate(g["llm_output"]):
        lg[0, u, vocab[w]] = 1.0
    toks = torch.tensor([[vocab[w] for w in g["tree_tokens"]]], dtype=torch.int32, device=DEV)
    spi.specinfer_verify_greedy(shape, lg, toks, tb.parent, tb.n_nodes, an, at, na, st.workspace)
    torch.cuda.synchronize()
    assert na.item() == 3
    assert an[0, :3].tolist() == g["expected_accepted_nodes"]
    assert [g["vocab"][t] for t in at[0, :3].tolist()] == g["expected_tokens"]
    # ties: all-zero logits -> token 0 everywhere
    lg.zero_()
    spi.specinfer_verify_greedy(shape, lg, toks, tb.parent, tb.n_nodes, an, at, na, st.workspace)
    torch.cuda.synchronize()
    assert at[0, 0].item() == 0 and na.item() == 1


def _mss_compare(got, ref, label=""):
    """Bit-exact up to requests whose FIRST divergent decision has an oracle margin < 1e-5, at most
    1e-4 of the requests, each printed (tests/mss_compare.py)."""
    return compare_sampled(got, ref, label=label)


@pytest.mark.parametrize("V,T", [(5, 1.0), (1000, 0.7), (32000, 1.0), (50272, 1.3)])
def test_verify_mss_parity(V, T):
    rng = np.random.default_rng(V + 1)
    B = 48
    trees = [W.random_tree(int(rng.integers(1, 40)), 8, 5, rng) for _ in range(B)]
    tb = W.make_tree_batch(trees, [3] * B, max_nodes=40, max_depth=8, device=DEV)
    shape, st, vi, outs = _verify_setup(tb, V, "mss", seed=V, Hq=1, Hkv=1)
    rids = torch.arange(1000, 1000 + B, dtype=torch.int32, device=DEV)
    spi.specinfer_verify_mss(shape, vi.logits, vi.tree_tokens, tb.parent, tb.n_nodes, vi.draft_probs, T, 1234,
                             17, rids, *outs, st.workspace)
    torch.cuda.synchronize()
    ref = oracle.verify_mss(vi.logits.cpu().numpy(), vi.tree_tokens.cpu().numpy(), tb.parent.cpu().numpy(),
                            tb.n_nodes.cpu().numpy(), vi.draft_probs.cpu().numpy(), temperature=T, seed=1234,
                            offset=17, request_ids=rids.cpu().numpy(), path_len=9)
    _mss_compare(outs, ref, f"mss V={V} T={T}")


def test_verify_mss_config_c4_full():
    """C4 (B=64, 233-node tree <8,4,1,...>, V=50272), full size, MSS."""
    cfg = W.CONFIGS["C4"]
    tb = W.config_tree_batch(cfg, device=DEV)
    shape, st, vi, outs = _verify_setup(tb, cfg.vocab, "mss", seed=cfg.seed, Hq=1, Hkv=1)
    spi.specinfer_verify_mss(shape, vi.logits, vi.tree_tokens, tb.parent, tb.n_nodes, vi.draft_probs, 1.0, 4, 0,
                             None, *outs, st.workspace)
    torch.cuda.synchronize()
    ref = oracle.verify_mss(vi.logits.cpu().numpy(), vi.tree_tokens.cpu().numpy(), tb.parent.cpu().numpy(),
                            tb.n_nodes.cpu().numpy(), vi.draft_probs.cpu().numpy(), seed=4, offset=0,
                            path_len=cfg.max_depth + 1)
    _mss_compare(outs, ref, "mss C4 full")


def test_verify_config_c2_full_greedy_and_mss():
    cfg = W.CONFIGS["C2"]
    tb = W.config_tree_batch(cfg, device=DEV)
    for mode in ("greedy", "mss"):
        shape, st, vi, (an, at, na) = _verify_setup(tb, cfg.vocab, mode, seed=cfg.seed)
        if mode == "greedy":
            spi.specinfer_verify_greedy(shape, vi.logits, vi.tree_tokens, tb.parent, tb.n_nodes, an, at, na,
                                        st.workspace)
            torch.cuda.synchronize()
            r = oracle.verify_greedy(vi.logits.cpu().numpy(), vi.tree_tokens.cpu().numpy(), tb.parent.cpu().numpy(),
                                     tb.n_nodes.cpu().numpy(), path_len=9)
            for x, y in zip(r, (an, at, na)):
                assert np.array_equal(x, y.cpu().numpy())
        else:
            spi.specinfer_verify_mss(shape, vi.logits, vi.tree_tokens, tb.parent, tb.n_nodes, vi.draft_probs, 1.0,
                                     2, 0, None, an, at, na, st.workspace)
            torch.cuda.synchronize()
            r = oracle.verify_mss(vi.logits.cpu().numpy(), vi.tree_tokens.cpu().numpy(), tb.parent.cpu().numpy(),
                                  tb.n_nodes.cpu().numpy(), vi.draft_probs.cpu().numpy(), seed=2, offset=0,
                                  path_len=9)
            _mss_compare((an, at, na), r, "mss C2 full")


def test_philox_kat_on_device(golden):
    g = golden("philox_kat.json")
    ck = torch.tensor([[int(x, 16) for x in v["ctr"] + v["key"]] for v in g["vectors"]], dtype=torch.int64,
                      device=DEV)
    out = spi.specinfer_philox_debug(ck).cpu().numpy()
    for row, v in zip(out, g["vectors"]):
        assert [f"{int(x):08x}" for x in row] == v["out"]


def test_verify_invalid_tree():
    tb = W.make_tree_batch([W.chain_tree(5), W.chain_tree(5)], [0, 0], device=DEV)
    tb.depth[0, 3] = 7   # depth mismatch
    shape, st, vi, (an, at, na) = _verify_setup(tb, 50, "greedy", seed=3)
    spi.specinfer_verify_greedy(shape, vi.logits, vi.tree_tokens, tb.parent, tb.n_nodes, an, at, na, st.workspace)
    torch.cuda.synchronize()
    assert na[0].item() == 0 and (an[0] == -1).all() and (at[0] == -1).all() and na[1].item() >= 1
    spi.specinfer_verify_mss(shape, vi.logits, vi.tree_tokens, tb.parent, tb.n_nodes, vi.draft_probs, 1.0, 1, 0,
                             None, an, at, na, st.workspace)
    torch.cuda.synchronize()
    assert na[0].item() == 0 and (an[0] == -1).all()
    assert spi.specinfer_read_device_status(st.workspace) & 1


# ---------------------------------------------------------------------------------------------
# KV commit
# ---------------------------------------------------------------------------------------------

@pytest.mark.parametrize("L,Hkv", [(1, 2), (3, 8)])
def test_kv_commit_parity(L, Hkv):
    rng = np.random.default_rng(L * 10 + Hkv)
    B = 9
    trees = [W.random_tree(int(rng.integers(1, 30)), 8, 3, rng) for _ in range(B)]
    pls = [int(x) for x in rng.integers(0, 100, B)]
    tb = W.make_tree_batch(trees, pls, max_nodes=30, max_depth=8, device=DEV)
    smax = max(pls) + 32
    ai = W.make_attention_inputs(tb, 1, Hkv, Hkv, smax, seed=9, device=DEV, cache_layers=L)
    shape = _shape(tb, Hkv, Hkv, smax, num_layers=L, vocab=64)
    st = spi.TreeState.create(shape, tb.parent, tb.depth, tb.prefix_len, tb.n_nodes)
    st.prepare()
    vi = W.make_verify_inputs(tb, 64, seed=5, mode="greedy", device=DEV, tau=0.05)
    an = torch.empty((B, 9), dtype=torch.int32, device=DEV)
    at, na = torch.empty_like(an), torch.empty((B,), dtype=torch.int32, device=DEV)
    spi.specinfer_verify_greedy(shape, vi.logits, vi.tree_tokens, tb.parent, tb.n_nodes, an, at, na, st.workspace)
    na[2] = 0   # a request with nothing accepted (e.g. invalid tree) is left alone
    k, v = ai.k_cache.clone(), ai.v_cache.clone()
    pl = tb.prefix_len.clone()
    spi.specinfer_kv_commit(shape, k, v, pl, an, na)
    torch.cuda.synchronize()
    kh = ai.k_cache.cpu().view(torch.int16).numpy().view(np.uint16).copy()
    vh = ai.v_cache.cpu().view(torch.int16).numpy().view(np.uint16).copy()
    plh = tb.prefix_len.cpu().numpy().copy()
    oracle.kv_commit(kh, vh, plh, an.cpu().numpy(), na.cpu().numpy())
    assert np.array_equal(plh, pl.cpu().numpy())
    kg = k.cpu().view(torch.int16).numpy().view(np.uint16)
    vg = v.cpu().view(torch.int16).numpy().view(np.uint16)
    for b in range(B):
        e = int(plh[b]) if na[b].item() > 0 else smax
        assert np.array_equal(kh[:, b, :, :e], kg[:, b, :, :e])
        assert np.array_equal(vh[:, b, :, :e], vg[:, b, :, :e])
    assert int(na.cpu().numpy()[[0, 1, 3]].max()) >= 2  # some request committed a moved path


@pytest.mark.parametrize("B,Hq,Hkv,expansion,P", [(2, 32, 32, (1, 1, 3, 1, 1, 1, 1, 1), 2048),   # split-KV
                                                  (6, 8, 8, (1, 2, 2), 3000),                    # stream-K
                                                  (3, 16, 2, (1, 2, 2, 2), 700),                 # rows kernel
                                                  (16, 32, 32, (1, 1, 3, 1, 1, 1, 1, 1), 600),   # dynamic items
                                                  (8, 64, 8, (1, 2, 2, 2, 2, 2), 500)])          # rows, dynamic
def test_attention_early_prefix_bit_identical(B, Hq, Hkv, expansion, P):
    """SPECINFER_ATTN_EARLY_PREFIX (committed-prefix tiles staged before the programmatic dependency
    resolves) on layers >= 1 of a CUDA-graph chain gives bit-identical outputs to plain launches,
    and matches the oracle."""
    parent, depth = W.expansion_tree(expansion)
    tb = W.make_tree_batch([(parent, depth)] * B, list(W.ragged_prefix(P, B)), device=DEV, max_depth=8)
    smax = P + tb.max_nodes + 2
    L = 4
    ai = W.make_attention_inputs(tb, L, Hq, Hkv, smax, seed=31, device=DEV, poison=True)
    shape = _shape(tb, Hq, Hkv, smax)
    outs = []
    for early in (False, True):
        st = spi.TreeState.create(shape, tb.parent, tb.depth, tb.prefix_len, tb.n_nodes)
        out = torch.full(ai.q.shape, float("nan"), dtype=torch.bfloat16, device=DEV)
        s = torch.cuda.Stream()
        s.wait_stream(torch.cuda.current_stream())
        with torch.cuda.stream(s):
            st.prepare()
            for l in range(L):
                st.attention(ai.q[l], ai.k_cache[l], ai.v_cache[l], out[l], prefetch=early and l > 0)
        torch.cuda.synchronize()
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g, stream=s):
            st.prepare()
            for l in range(L):
                st.attention(ai.q[l], ai.k_cache[l], ai.v_cache[l], out[l], prefetch=early and l > 0)
        out.fill_(float("nan"))
        g.replay()
        g.replay()
        torch.cuda.synchronize()
        outs.append(out)
    n = tb.n_nodes.cpu().numpy()
    for b in range(B):
        assert torch.equal(outs[0][:, b, :n[b]], outs[1][:, b, :n[b]])
    bs = None if B <= 6 else [0, B // 2, B - 1]
    _check_rows(outs[1][L - 1], _oracle_attention(ai, tb, layer=L - 1, bs=bs), tb, bs=bs)
