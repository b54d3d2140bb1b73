"""GPU parity of the NEXT-3 naive-sampling verifier against the fp64 oracle:
bit-exact except race decisions whose relative margin is below 1e-5 (the GPU draws in fp32 /
MUFU log2), plus the shared-counter contract with MSS at leaves."""
import numpy as np
import pytest
import torch

import oracle
import workloads as W
from tests.test_gpu_parity import DEV, _mss_compare, _verify_setup

pytestmark = pytest.mark.gpu

if torch.cuda.is_available():
    import paper_conf_asplos_miaoozcwzwzyssc24_b200 as spi


@pytest.mark.parametrize("V,T", [(5, 1.0), (1001, 0.7), (32000, 1.0), (50272, 1.3)])
def test_verify_ns_parity(V, T):
    rng = np.random.default_rng(V + 7)
    B = 48
    trees = [W.random_tree(int(rng.integers(1, 40)), 8, 5, rng) for _ in range(B)]
    tb = W.make_tree_batch(trees, [3] * B, max_nodes=40, max_depth=8, device=DEV)
    shape, st, vi, outs = _verify_setup(tb, V, "mss", seed=V, Hq=1, Hkv=1)
    rids = torch.arange(500, 500 + B, dtype=torch.int32, device=DEV)
    spi.specinfer_verify_ns(shape, vi.logits, vi.tree_tokens, tb.parent, tb.n_nodes, T, 99, 5, rids, *outs,
                            st.workspace)
    torch.cuda.synchronize()
    ref = oracle.verify_ns(vi.logits.cpu().numpy(), vi.tree_tokens.cpu().numpy(), tb.parent.cpu().numpy(),
                           tb.n_nodes.cpu().numpy(), temperature=T, seed=99, offset=5,
                           request_ids=rids.cpu().numpy(), path_len=9)
    _mss_compare(outs, ref, f"ns V={V} T={T}")


def test_verify_ns_config_c2_full_and_leaf_contract():
    """C2 at full size; and on root-only trees NS and MSS draw the same token (same counters)."""
    cfg = W.CONFIGS["C2"]
    tb = W.config_tree_batch(cfg, device=DEV)
    shape, st, vi, (an, at, na) = _verify_setup(tb, cfg.vocab, "mss", seed=cfg.seed)
    spi.specinfer_verify_ns(shape, vi.logits, vi.tree_tokens, tb.parent, tb.n_nodes, 1.0, 2, 0, None, an, at, na,
                            st.workspace)
    torch.cuda.synchronize()
    ref = oracle.verify_ns(vi.logits.cpu().numpy(), vi.tree_tokens.cpu().numpy(), tb.parent.cpu().numpy(),
                           tb.n_nodes.cpu().numpy(), seed=2, offset=0, path_len=cfg.max_depth + 1)
    _mss_compare((an, at, na), ref, "ns C2 full")
    B = 32
    tb1 = W.make_tree_batch([W.chain_tree(1)] * B, [0] * B, max_depth=8, device=DEV)
    shape1, st1, vi1, o1 = _verify_setup(tb1, 4096, "mss", seed=5)
    o2 = [torch.empty_like(x) for x in o1]
    spi.specinfer_verify_ns(shape1, vi1.logits, vi1.tree_tokens, tb1.parent, tb1.n_nodes, 1.0, 3, 1, None, *o1,
                            st1.workspace)
    spi.specinfer_verify_mss(shape1, vi1.logits, vi1.tree_tokens, tb1.parent, tb1.n_nodes, vi1.draft_probs, 1.0, 3, 1,
                             None, *o2, st1.workspace)
    torch.cuda.synchronize()
    for x, y in zip(o1, o2):
        assert torch.equal(x, y)


def test_verify_ns_invalid_tree():
    tb = W.make_tree_batch([W.chain_tree(5), W.chain_tree(5)], [0, 0], device=DEV)
    tb.depth[0, 3] = 7   # depth mismatch
    shape, st, vi, (an, at, na) = _verify_setup(tb, 50, "mss", seed=3)
    spi.specinfer_verify_ns(shape, vi.logits, vi.tree_tokens, tb.parent, tb.n_nodes, 1.0, 1, 0, None, an, at, na,
                            st.workspace)
    torch.cuda.synchronize()
    assert na[0].item() == 0 and (an[0] == -1).all() and na[1].item() >= 1
