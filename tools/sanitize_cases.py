"""Small launches of every hand-written synchronisation protocol, for compute-sanitizer
(memcheck / racecheck / synccheck) runs under gpurun:

  * C1 (one request, 16-node tree, swapped kernel, whole-unit schedule);
  * tiny random trees (ragged n, P around tile boundaries, NT = 16 / 32 / 64);
  * the split-KV cluster mode (batch 1, P = 2048: DSMEM push + cluster merge);
  * stream-K split items, both merge paths (staged: <= 8 pieces; batched: one long request);
  * the rows-as-M kernel (G * Nmax > 64: lock-step lanes);
  * verify_greedy (last-CTA walk), verify_mss (8-CTA cluster, DSMEM reductions), verify_ns, kv_commit.

Each case checks its result against the oracle so a sanitizer run is also a parity run.

    compute-sanitizer --tool racecheck python tools/sanitize_cases.py [--only NAME]
"""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import oracle
import paper_conf_asplos_miaoozcwzwzyssc24_b200 as spi
import workloads as W

DEV = "cuda:0"


def attention_case(trees, pls, Hq, Hkv, name, max_depth=8):
    tb = W.make_tree_batch(trees, pls, device=DEV, max_depth=max_depth)
    smax = max(pls) + tb.max_nodes + 2
    ai = W.make_attention_inputs(tb, 1, Hq, Hkv, smax, seed=5, device=DEV, poison=True)
    shape = spi.make_shape(tb.parent.shape[0], tb.max_nodes, Hq, Hkv, smax, max_depth=max_depth)
    st = spi.TreeState.create(shape, tb.parent, tb.depth, tb.prefix_len, tb.n_nodes)
    st.prepare()
    out = torch.full(ai.q.shape[1:], float("nan"), dtype=torch.bfloat16, device=DEV)
    st.attention(ai.q[0], ai.k_cache[0], ai.v_cache[0], out)
    torch.cuda.synchronize()
    ref = oracle.tree_attention(ai.q[0].cpu(), ai.k_cache[0].cpu(), ai.v_cache[0].cpu(), tb.parent.cpu(),
                                tb.depth.cpu(), tb.prefix_len.cpu(), tb.n_nodes.cpu())
    n = tb.n_nodes.cpu().numpy()
    err = max(float(np.abs(out[b, :n[b]].float().cpu().numpy() - ref[b, :n[b]]).max()) for b in range(len(n)))
    assert err <= 1e-2, (name, err)
    print(f"{name}: ok (max |err| {err:.2e})", flush=True)


def case_c1():
    p, d = W.expansion_tree((1, 2, 2, 2))
    attention_case([(p, d)], [128], 32, 32, "C1")


def case_tiny():
    rng = np.random.default_rng(3)
    for Hq, Hkv, N in ((2, 2, 8), (4, 2, 16), (4, 4, 64)):
        trees = [W.random_tree(int(rng.integers(1, N + 1)), 8, 4, rng) for _ in range(3)]
        attention_case(trees, [0, 127, 300], Hq, Hkv, f"tiny Hq{Hq} Hkv{Hkv} N{N}")


def case_splitkv():
    p, d = W.expansion_tree((1, 1, 3, 1, 1, 1, 1, 1))
    attention_case([(p, d)], [2048], 4, 4, "split-KV cluster (B 1, P 2048)")


def case_streamk():
    p, d = W.expansion_tree((1, 1, 3, 1, 1, 1, 1, 1))
    attention_case([(p, d)] * 3, list(W.ragged_prefix(3000, 3)), 8, 8, "stream-K staged merge")
    p, d = W.expansion_tree((1, 2, 2))
    attention_case([(p, d)] * 40, [40000] + [5 + 3 * b for b in range(39)], 2, 1, "stream-K batched merge")


def case_rows():
    p, d = W.expansion_tree((1, 2, 2, 2))
    attention_case([(p, d)] * 3, [700, 650, 130], 16, 2, "rows kernel (G 8, 15 nodes)")


def case_verify():
    rng = np.random.default_rng(7)
    B, V = 12, 3000
    trees = [W.random_tree(int(rng.integers(1, 30)), 8, 4, rng) for _ in range(B)]
    tb = W.make_tree_batch(trees, [3] * B, max_nodes=30, max_depth=8, device=DEV)
    shape = spi.make_shape(B, 30, 1, 1, 40, vocab=V, max_depth=8, num_layers=2)
    st = spi.TreeState.create(shape, tb.parent, tb.depth, tb.prefix_len, tb.n_nodes)
    st.prepare()
    vi = W.make_verify_inputs(tb, V, seed=2, mode="mss", device=DEV)
    outs = [torch.empty((B, 9), dtype=torch.int32, device=DEV), torch.empty((B, 9), dtype=torch.int32, device=DEV),
            torch.empty((B,), dtype=torch.int32, device=DEV)]
    spi.specinfer_verify_greedy(shape, vi.logits, vi.tree_tokens, tb.parent, tb.n_nodes, *outs, st.workspace)
    torch.cuda.synchronize()
    r = oracle.verify_greedy(vi.logits.cpu().numpy(), vi.tree_tokens.cpu().numpy(), tb.parent.cpu().numpy(),
                             tb.n_nodes.cpu().numpy(), path_len=9)
    assert all(np.array_equal(a, b.cpu().numpy()) for a, b in zip(r, outs))
    print("verify_greedy: ok", flush=True)
    spi.specinfer_verify_mss(shape, vi.logits, vi.tree_tokens, tb.parent, tb.n_nodes, vi.draft_probs, 1.0, 9, 1,
                             None, *outs, st.workspace)
    torch.cuda.synchronize()
    r = oracle.verify_mss(vi.logits.cpu().numpy(), vi.tree_tokens.cpu().numpy(), tb.parent.cpu().numpy(),
                          tb.n_nodes.cpu().numpy(), vi.draft_probs.cpu().numpy(), seed=9, offset=1, path_len=9)
    assert all(np.array_equal(a, b.cpu().numpy()) for a, b in zip(r[:3], outs))
    print("verify_mss: ok", flush=True)
    spi.specinfer_verify_ns(shape, vi.logits, vi.tree_tokens, tb.parent, tb.n_nodes, 1.0, 9, 1, None, *outs,
                            st.workspace)
    torch.cuda.synchronize()
    r = oracle.verify_ns(vi.logits.cpu().numpy(), vi.tree_tokens.cpu().numpy(), tb.parent.cpu().numpy(),
                         tb.n_nodes.cpu().numpy(), seed=9, offset=1, path_len=9)
    assert all(np.array_equal(a, b.cpu().numpy()) for a, b in zip(r[:3], outs))
    print("verify_ns: ok", flush=True)
    ai = W.make_attention_inputs(tb, 1, 2, 2, 40, seed=3, device=DEV, cache_layers=2)
    k, v, pl = ai.k_cache.clone(), ai.v_cache.clone(), tb.prefix_len.clone()
    shape2 = spi.make_shape(B, 30, 2, 2, 40, vocab=V, max_depth=8, num_layers=2)
    spi.specinfer_kv_commit(shape2, k, v, pl, outs[0], outs[2])
    torch.cuda.synchronize()
    kh = ai.k_cache.cpu().view(torch.int16).numpy().view(np.uint16).copy()
    vh = ai.v_cache.cpu().view(torch.int16).numpy().view(np.uint16).copy()
    plh = tb.prefix_len.cpu().numpy().copy()
    oracle.kv_commit(kh, vh, plh, outs[0].cpu().numpy(), outs[2].cpu().numpy())
    kg = k.cpu().view(torch.int16).numpy().view(np.uint16)
    assert np.array_equal(plh, pl.cpu().numpy())
    assert all(np.array_equal(kg[:, b, :, :plh[b]], kh[:, b, :, :plh[b]]) for b in range(B))
    print("kv_commit: ok", flush=True)


CASES = {"c1": case_c1, "tiny": case_tiny, "splitkv": case_splitkv, "streamk": case_streamk, "rows": case_rows,
         "verify": case_verify}

if __name__ == "__main__":
    ap = argparse.ArgumentParser()
    ap.add_argument("--only", default=None, choices=sorted(CASES))
    ap.add_argument("--lib", default=None, help="A/B: load another build of libspecinfer.so")
    a = ap.parse_args()
    if a.lib:
        spi.load_library(a.lib)
    for name, fn in CASES.items():
        if a.only is None or a.only == name:
            fn()
