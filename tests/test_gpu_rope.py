"""GPU parity of NEXT-4's tree position encoding (specinfer_tree_rope, reading A4: node i at position
P_b + depth[i]) against the oracle (oracle.tree_rope, pinned in tests/test_oracle_rope.py).

Bar: every rotated element within one bf16 rounding of the fp64 oracle (the CUDA path rotates in
fp32 on the same fp32 angle fp32(pos) * fp32(theta_d), then rounds once to bf16):
|gpu - ref| <= 2^-8 |ref| + 2^-20 (|x_d| + |x_{d+64}|).  Rows / slots outside the tree bit-identical.
End to end: tree attention of the rotated tree within the attention bar (1e-2 / 1e-3).
"""
import numpy as np
import pytest
import torch

import oracle
import workloads as W

pytestmark = pytest.mark.gpu

if torch.cuda.is_available():
    import paper_conf_asplos_miaoozcwzwzyssc24_b200 as spi

DEV = "cuda:0"
D = 128


def _setup(Hq, Hkv, Nmax, P, seed):
    rng = np.random.default_rng(seed)
    B = 3
    trees = [W.random_tree(int(rng.integers(1, Nmax + 1)), 8, 4, rng) for _ in range(B)]
    pls = [P, max(P - 37, 0), P + 5]
    tb = W.make_tree_batch(trees, pls, max_nodes=Nmax, max_depth=8, device=DEV)
    smax = max(pls) + Nmax + 3
    ai = W.make_attention_inputs(tb, 1, Hq, Hkv, smax, seed=seed, device=DEV)
    shape = spi.make_shape(B, Nmax, Hq, Hkv, smax, max_depth=8)
    return tb, ai, shape


def _bound(ref, raw):
    # one bf16 rounding of the result + fp32 arithmetic on the pair
    pair = np.abs(raw) + np.abs(np.concatenate([raw[..., D // 2:], raw[..., :D // 2]], axis=-1))
    return 2.0 ** -8 * np.abs(ref) + 2.0 ** -20 * pair + 1e-30


@pytest.mark.parametrize("Hq,Hkv,Nmax,P", [(8, 2, 40, 300), (4, 4, 16, 0), (32, 32, 21, 2048), (8, 8, 64, 8000)])
def test_tree_rope_parity(Hq, Hkv, Nmax, P):
    tb, ai, shape = _setup(Hq, Hkv, Nmax, P, seed=Nmax + P)
    q0, k0 = ai.q[0].clone(), ai.k_cache[0].clone()
    q, k = ai.q[0], ai.k_cache[0]
    spi.specinfer_tree_rope(shape, q, k, tb.prefix_len, tb.depth, tb.n_nodes, 10000.0)
    torch.cuda.synchronize()
    pl, nn_, dep = tb.prefix_len.cpu().numpy(), tb.n_nodes.cpu().numpy(), tb.depth.cpu().numpy()
    q_raw, k_raw = q0.float().cpu().numpy(), k0.float().cpu().numpy()
    q_ref, k_ref = oracle.tree_rope(q_raw, k_raw, pl, dep, nn_)
    qg, kg = q.float().cpu().numpy(), k.float().cpu().numpy()
    for b in range(q.shape[0]):
        n, p = int(nn_[b]), int(pl[b])
        e = np.abs(qg[b, :n] - q_ref[b, :n])
        assert np.all(e <= _bound(q_ref[b, :n], q_raw[b, :n])), (b, e.max())
        e = np.abs(kg[b, :, p:p + n] - k_ref[b, :, p:p + n])
        assert np.all(e <= _bound(k_ref[b, :, p:p + n], k_raw[b, :, p:p + n])), (b, e.max())
        # outside the tree: untouched (bitwise)
        assert torch.equal(q[b, n:], q0[b, n:])
        assert torch.equal(k[b, :, :p], k0[b, :, :p]) and torch.equal(k[b, :, p + n:], k0[b, :, p + n:])


def test_tree_rope_queries_only_and_keys_only():
    tb, ai, shape = _setup(8, 2, 24, 100, seed=3)
    q0, k0 = ai.q[0].clone(), ai.k_cache[0].clone()
    spi.specinfer_tree_rope(shape, ai.q[0], None, tb.prefix_len, tb.depth, tb.n_nodes)
    torch.cuda.synchronize()
    assert torch.equal(ai.k_cache[0], k0) and not torch.equal(ai.q[0], q0)
    q1 = ai.q[0].clone()
    spi.specinfer_tree_rope(shape, None, ai.k_cache[0], tb.prefix_len, tb.depth, tb.n_nodes)
    torch.cuda.synchronize()
    assert torch.equal(ai.q[0], q1) and not torch.equal(ai.k_cache[0], k0)
    with pytest.raises(ValueError):
        spi.specinfer_tree_rope(shape, None, None, tb.prefix_len, tb.depth, tb.n_nodes)


@pytest.mark.parametrize("Hq,Hkv,Nmax", [(8, 2, 40), (2, 2, 100)])
def test_tree_rope_then_attention(Hq, Hkv, Nmax):
    """rope (P_b + depth) -> tree attention on the GPU vs oracle.tree_rope -> oracle.tree_attention."""
    P = 500
    tb, ai, shape = _setup(Hq, Hkv, Nmax, P, seed=11 + Nmax)
    pl, nn_, dep = tb.prefix_len.cpu().numpy(), tb.n_nodes.cpu().numpy(), tb.depth.cpu().numpy()
    q_ref, k_ref = oracle.tree_rope(ai.q[0].float().cpu().numpy(), ai.k_cache[0].float().cpu().numpy(), pl, dep, nn_)
    spi.specinfer_tree_rope(shape, ai.q[0], ai.k_cache[0], tb.prefix_len, tb.depth, tb.n_nodes)
    st = spi.TreeState.create(shape, tb.parent, tb.depth, tb.prefix_len, tb.n_nodes)
    st.prepare()
    out = torch.empty_like(ai.q[0])
    st.attention(ai.q[0], ai.k_cache[0], ai.v_cache[0], out)
    torch.cuda.synchronize()
    bf = lambda a: torch.as_tensor(np.asarray(a, np.float32)).to(torch.bfloat16)
    ref = oracle.tree_attention(bf(q_ref), bf(k_ref), ai.v_cache[0].cpu(), tb.parent.cpu(), tb.depth.cpu(),
                                tb.prefix_len.cpu(), tb.n_nodes.cpu())
    errs = []
    for b in range(out.shape[0]):
        n = int(nn_[b])
        errs.append(np.abs(out[b, :n].float().cpu().numpy() - ref[b, :n]).reshape(-1))
    e = np.concatenate(errs)
    assert e.max() <= 1e-2 and e.mean() <= 1e-3, (e.max(), e.mean())


def test_rope_then_commit_keeps_slot_positions():
    """R29: after the tree is encoded at P_b + depth[i] and the accepted path is committed, every
    committed slot P + j holds a key encoded at position P + j (path[j] has depth j), so the cache
    stays a plain position-encoded sequence.  Checked against oracle.rope_rotate of the raw keys."""
    rng = np.random.default_rng(21)
    B, Hq, Hkv, Nmax, P = 3, 8, 4, 24, 257
    trees = [W.random_tree(Nmax, 8, 3, rng) for _ in range(B)]
    tb = W.make_tree_batch(trees, [P, P - 40, P + 9], max_nodes=Nmax, max_depth=8, device=DEV)
    smax = P + 9 + Nmax + 3
    ai = W.make_attention_inputs(tb, 1, Hq, Hkv, smax, seed=21, device=DEV)
    shape = spi.make_shape(B, Nmax, Hq, Hkv, smax, max_depth=8)
    k_raw = ai.k_cache[0].float().cpu().numpy()
    spi.specinfer_tree_rope(shape, None, ai.k_cache[0], tb.prefix_len, tb.depth, tb.n_nodes)
    # accepted path: root -> deepest-first-child chain (a valid root path of each tree)
    par = tb.parent.cpu().numpy()
    nn_ = tb.n_nodes.cpu().numpy()
    paths = np.zeros((B, 9), np.int32)
    n_acc = np.zeros(B, np.int32)
    for b in range(B):
        path = [0]
        while True:
            kids = [c for c in range(1, nn_[b]) if par[b, c] == path[-1]]
            if not kids:
                break
            path.append(kids[-1])
        paths[b, :len(path)] = path
        n_acc[b] = len(path)
    pl = tb.prefix_len.clone()
    spi.specinfer_kv_commit(shape, ai.k_cache, ai.v_cache, pl, torch.from_numpy(paths).to(DEV),
                            torch.from_numpy(n_acc).to(DEV))
    torch.cuda.synchronize()
    kg = ai.k_cache[0].float().cpu().numpy()
    p0 = tb.prefix_len.cpu().numpy()
    for b in range(B):
        for j in range(n_acc[b]):
            slot = int(p0[b]) + j
            want = oracle.rope_rotate(k_raw[b, :, int(p0[b]) + paths[b, j]], np.full(Hkv, slot))
            got = kg[b, :, slot]
            raw = k_raw[b, :, int(p0[b]) + paths[b, j]]
            assert np.all(np.abs(got - want) <= _bound(want, raw)), (b, j)
    assert np.array_equal(pl.cpu().numpy(), p0 + n_acc)
