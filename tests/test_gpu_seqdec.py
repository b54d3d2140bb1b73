"""GPU parity of the NEXT-1 sequence-based decoding baseline (§4.2, Fig. 4
left L682): specinfer_leaf_paths bit-exact against the oracle's decomposition, and the packed
per-sequence caches run through specinfer_tree_attention (chain trees, one launch for all
sequences or one launch per sequence) reproduce the oracle's tree attention at every node of
every sequence (same tolerance as tree attention)."""
import numpy as np
import pytest
import torch

import oracle
import workloads as W
from tests.test_gpu_parity import DEV, MAX_ABS, MEAN_ABS, _oracle_attention, _shape

pytestmark = pytest.mark.gpu

if torch.cuda.is_available():
    import paper_conf_asplos_miaoozcwzwzyssc24_b200 as spi


def _leaf_paths_gpu(tb, Hq=2, Hkv=2):
    shape = _shape(tb, Hq, Hkv, int(tb.prefix_len.max()) + tb.max_nodes)
    B, N, Lp = tb.parent.shape[0], tb.max_nodes, tb.max_depth + 1
    paths = torch.empty((B, N, Lp), dtype=torch.int32, device=DEV)
    plen = torch.empty((B, N), dtype=torch.int32, device=DEV)
    nl = torch.empty((B,), dtype=torch.int32, device=DEV)
    ws = spi.alloc_workspace(shape, DEV)
    ws.zero_()
    spi.specinfer_leaf_paths(shape, tb.parent, tb.n_nodes, paths, plen, nl, ws)
    bits = spi.specinfer_read_device_status(ws)
    return paths.cpu().numpy(), plen.cpu().numpy(), nl.cpu().numpy(), bits


@pytest.mark.parametrize("Nmax", [1, 8, 33, 256])
def test_leaf_paths_parity(Nmax):
    rng = np.random.default_rng(Nmax)
    B = 6
    trees = [W.random_tree(int(rng.integers(1, Nmax + 1)), 8, 5, rng) for _ in range(B)]
    tb = W.make_tree_batch(trees, [4] * B, max_nodes=Nmax, max_depth=8, device=DEV)
    paths, plen, nl, bits = _leaf_paths_gpu(tb)
    assert bits == 0
    ref = oracle.leaf_paths(tb.parent.cpu().numpy(), tb.n_nodes.cpu().numpy())
    for b in range(B):
        assert nl[b] == len(ref[b])
        for r, pth in enumerate(ref[b]):
            assert plen[b, r] == len(pth)
            assert list(paths[b, r, :len(pth)]) == pth
            assert np.all(paths[b, r, len(pth):] == -1)
        assert np.all(plen[b, nl[b]:] == 0)


def test_leaf_paths_fig4_and_invalid(golden):
    g = golden("fig4_mask.json")
    par = np.asarray(g["parent"], np.int32)
    bad = par.copy()
    bad[3] = 7  # parent after child: invalid
    dep = np.zeros_like(par)
    for i in range(1, len(par)):
        dep[i] = dep[par[i]] + 1
    tb = W.make_tree_batch([(par, dep), (bad, dep)], [0, 0], max_depth=8, device=DEV)
    paths, plen, nl, bits = _leaf_paths_gpu(tb)
    assert nl[0] == 3 and plen[0, :3].sum() == g["sequence_query_rows"]
    assert nl[1] == 0 and bits & 1


@pytest.mark.parametrize("Hq,Hkv,P,per_seq", [(4, 4, 300, False), (8, 2, 129, False), (2, 2, 0, True),
                                              (32, 32, 512, False)])
def test_sequence_baseline_matches_tree_attention(Hq, Hkv, P, per_seq):
    rng = np.random.default_rng(P + Hq)
    B, Nmax = 3, 24
    trees = [W.random_tree(int(rng.integers(1, Nmax + 1)), 8, 4, rng) for _ in range(B)]
    pls = [P, max(P - 3, 0), P + 7]
    tb = W.make_tree_batch(trees, pls, max_nodes=Nmax, max_depth=8, device=DEV)
    smax = max(pls) + Nmax + 2
    ai = W.make_attention_inputs(tb, 1, Hq, Hkv, smax, seed=P + 1, device=DEV, poison=True)
    shape = _shape(tb, Hq, Hkv, smax)
    sb = spi.SequenceBaseline(shape, tb.parent, tb.depth, tb.prefix_len, tb.n_nodes)
    sb.build(ai.q[0], ai.k_cache[0], ai.v_cache[0])
    out = sb.attention(per_sequence=per_seq).float().cpu().numpy()
    torch.cuda.synchronize()
    ref = _oracle_attention(ai, tb)
    paths = oracle.leaf_paths(tb.parent.cpu().numpy(), tb.n_nodes.cpu().numpy())
    errs = []
    s = 0
    for b in range(B):
        for pth in paths[b]:
            e = np.abs(out[s, :len(pth)] - ref[b, pth])
            assert np.all(np.isfinite(out[s, :len(pth)]))
            errs.append(e.reshape(-1))
            s += 1
    assert s == sb.num_seqs
    e = np.concatenate(errs)
    assert e.max() <= MAX_ABS and e.mean() <= MEAN_ABS, (e.max(), e.mean())
