"""World-size-2 gloo test of the multi-GPU host logic (request sharding, global request ids, the
tokens-only all-gather).  The per-rank "device" work is the oracle, so this runs on CPU; the
invariant checked is that the gathered results equal a single-process run on the whole batch
(integer outputs bit-identical across world sizes)."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.multiprocessing as mp

import oracle
import workloads as W
from paper_conf_asplos_miaoozcwzwzyssc24_b200 import dist as D


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _inputs():
    rng = np.random.default_rng(0)
    B, N, V = 10, 24, 40
    trees = [W.random_tree(int(rng.integers(1, N + 1)), 8, 4, rng) for _ in range(B)]
    tb = W.make_tree_batch(trees, [3] * B, max_nodes=N, max_depth=8)
    vi = W.make_verify_inputs(tb, V, seed=3, mode="mss")
    return tb, vi


def _verify(tb, vi, lo, cnt):
    sl = slice(lo, lo + cnt)
    an, at, na, _ = oracle.verify_mss(vi.logits[sl].numpy(), vi.tree_tokens[sl].numpy(), tb.parent[sl].numpy(),
                                      tb.n_nodes[sl].numpy(), vi.draft_probs[sl].numpy(), seed=9, offset=2,
                                      request_ids=np.arange(lo, lo + cnt, dtype=np.int32), path_len=9)
    return torch.from_numpy(na), torch.from_numpy(at), torch.from_numpy(an)


def _worker(rank, world, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    torch.distributed.init_process_group("gloo", rank=rank, world_size=world)
    try:
        tb, vi = _inputs()
        B = tb.parent.shape[0]
        lo, cnt = D.shard_requests(B, world, rank)
        assert cnt == B // world  # equal shards for the gather
        na, at, an = _verify(tb, vi, lo, cnt)
        packed = D.pack_accepted(na, at, an)
        gathered = D.gather_accepted(packed)
        if rank == 0:
            q.put(gathered.numpy())
    finally:
        torch.distributed.destroy_process_group()


def test_sharding_math():
    assert D.shard_requests(10, 3, 0) == (0, 4)
    assert D.shard_requests(10, 3, 1) == (4, 3)
    assert D.shard_requests(10, 3, 2) == (7, 3)
    assert sum(D.shard_requests(17, 4, r)[1] for r in range(4)) == 17


def test_two_rank_gather_equals_single_process():
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    gathered = q.get(timeout=120)
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    tb, vi = _inputs()
    na, at, an = _verify(tb, vi, 0, tb.parent.shape[0])
    ref = D.pack_accepted(na, at, an).numpy()
    assert np.array_equal(gathered, ref)


# ---------------------------------------------------------------------------------------------
# kv-head sharding (GQA, C3): attention + commit on head shards of every request, verification
# request-sharded, one gather; the result must equal a single-process run
# ---------------------------------------------------------------------------------------------

def _kv_inputs():
    rng = np.random.default_rng(5)
    B, N, V, Hq, Hkv, P = 4, 12, 30, 8, 4, 9
    trees = [W.random_tree(int(rng.integers(2, N + 1)), 6, 3, rng) for _ in range(B)]
    tb = W.make_tree_batch(trees, [P] * B, max_nodes=N, max_depth=6)
    ai = W.make_attention_inputs(tb, 1, Hq, Hkv, P + N, seed=4)
    vi = W.make_verify_inputs(tb, V, seed=6, mode="greedy")
    return tb, ai, vi, Hq, Hkv


def _kv_worker(rank, world, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    torch.distributed.init_process_group("gloo", rank=rank, world_size=world)
    try:
        tb, ai, vi, Hq, Hkv = _kv_inputs()
        B = tb.parent.shape[0]
        kv0, nkv, q0, nq = D.shard_kv_heads(Hq, Hkv, world, rank)
        # attention on this rank's head shard of every request
        out = oracle.tree_attention(ai.q[0][:, :, q0:q0 + nq], ai.k_cache[0][:, kv0:kv0 + nkv],
                                    ai.v_cache[0][:, kv0:kv0 + nkv], tb.parent, tb.depth, tb.prefix_len, tb.n_nodes)
        # verification on this rank's requests
        lo, cnt = D.shard_requests(B, world, rank)
        sl = slice(lo, lo + cnt)
        an, at, na = oracle.verify_greedy(vi.logits[sl].numpy(), vi.tree_tokens[sl].numpy(),
                                          tb.parent[sl].numpy(), tb.n_nodes[sl].numpy(), path_len=7)
        g = D.gather_accepted(D.pack_accepted(torch.from_numpy(na), torch.from_numpy(at), torch.from_numpy(an)))
        na_all, _, an_all = D.unpack_accepted(g)
        # commit this rank's head shard of every request
        k = ai.k_cache[:, :, kv0:kv0 + nkv].contiguous().view(torch.int16).numpy().astype(np.uint16)
        v = ai.v_cache[:, :, kv0:kv0 + nkv].contiguous().view(torch.int16).numpy().astype(np.uint16)
        pl = tb.prefix_len.numpy().copy()
        oracle.kv_commit(k, v, pl, an_all.contiguous().numpy(), na_all.contiguous().numpy())
        q.put((rank, out, k, pl))
    finally:
        torch.distributed.destroy_process_group()


def test_two_rank_kv_head_sharding_equals_single_process():
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_kv_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = dict((r, (o, k, pl)) for r, o, k, pl in [q.get(timeout=120) for _ in range(world)])
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    tb, ai, vi, Hq, Hkv = _kv_inputs()
    out = oracle.tree_attention(ai.q[0], ai.k_cache[0], ai.v_cache[0], tb.parent, tb.depth, tb.prefix_len,
                                tb.n_nodes)
    an, at, na = oracle.verify_greedy(vi.logits.numpy(), vi.tree_tokens.numpy(), tb.parent.numpy(),
                                      tb.n_nodes.numpy(), path_len=7)
    k = ai.k_cache.contiguous().view(torch.int16).numpy().astype(np.uint16)
    v = ai.v_cache.contiguous().view(torch.int16).numpy().astype(np.uint16)
    pl = tb.prefix_len.numpy().copy()
    oracle.kv_commit(k, v, pl, an, na)
    n = tb.n_nodes.numpy()
    for r in range(world):
        kv0, nkv, q0, nq = D.shard_kv_heads(Hq, Hkv, world, r)
        o, kr, plr = res[r]
        for b in range(len(n)):
            np.testing.assert_array_equal(o[b, :n[b]], out[b, :n[b], q0:q0 + nq])
            assert np.array_equal(kr[:, b, :, :plr[b]], k[:, b, kv0:kv0 + nkv, :pl[b]])
        assert np.array_equal(plr, pl)


def test_bench_reference_arm_two_ranks_prints_one_line():
    """`bench.py --impl reference` under torchrun at N = 2 (the driver's launch): rank 0 alone
    times the oracle and prints ONE JSON line with the reference-arm keys; rank 1 exits 0."""
    import json
    import subprocess
    import sys

    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "2",
           "--master-addr", "127.0.0.1", "--master-port", str(_free_port()), "bench.py",
           "--impl", "reference", "--gpus", "2", "--steps", "1", "--warmup", "0", "--config", "C1"]
    r = subprocess.run(cmd, cwd=root, capture_output=True, text=True, timeout=300)
    assert r.returncode == 0, r.stderr[-2000:]
    lines = [l for l in r.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1, r.stdout
    d = json.loads(lines[0])
    assert d["impl"] == "reference" and d["n_gpus"] == 2 and d["steps"] == 1
    assert d["value"] > 0 and d["higher_is_better"] is True
    assert d["cpu_baseline"]["kind"] == "oracle" and d["cpu_baseline"]["value"] == d["value"]
    assert d["e2e"] == {"value": d["value"], "unit": d["unit"], "h2d_bytes_per_step": 0,
                        "d2h_bytes_per_step": 0}


# ---------------------------------------------------------------------------------------------
# the bench's step plumbing (paper_conf_asplos_miaoozcwzwzyssc24_b200/step.py + bench.Workload)
# end to end at world size 2 under gloo, with the oracle standing in for the device calls: both
# layouts, an uneven request split (5 requests over 2 ranks), strong scaling; every rank's accepted
# paths, attention outputs and committed cache equal the world-size-1 run's share bit for bit
# ---------------------------------------------------------------------------------------------

class OracleOps:
    """Host stand-in for step.DeviceOps (same call signatures) backed by the fp64 oracle."""

    class St:
        def __init__(self, shape, parent, depth, prefix_len, n_nodes):
            self.shape, self.parent, self.depth, self.prefix_len, self.n_nodes = shape, parent, depth, prefix_len, n_nodes

    def state(self, shape, parent, depth, prefix_len, n_nodes):
        return self.St(shape, parent, depth, prefix_len, n_nodes)

    def prepare(self, st):
        pass

    def attention(self, st, q, k, v, out, prefetch):
        r = oracle.tree_attention(q, k, v, st.parent, st.depth, st.prefix_len, st.n_nodes)
        out.copy_(torch.from_numpy(np.nan_to_num(r)).to(torch.bfloat16))

    def verify_greedy(self, shape, st, logits, tokens, parent, n_nodes, an, at, na):
        r = oracle.verify_greedy(logits.numpy(), tokens.numpy(), parent.numpy(), n_nodes.numpy(), path_len=an.shape[1])
        for dst, src in zip((an, at, na), r):
            dst.copy_(torch.from_numpy(src))

    def verify_mss(self, shape, st, logits, tokens, parent, n_nodes, draft, temperature, seed, offset, rids, an, at, na):
        r = oracle.verify_mss(logits.numpy(), tokens.numpy(), parent.numpy(), n_nodes.numpy(), draft.numpy(),
                              temperature=temperature, seed=seed, offset=offset, request_ids=rids.numpy(),
                              path_len=an.shape[1])
        for dst, src in zip((an, at, na), r[:3]):
            dst.copy_(torch.from_numpy(src))

    def kv_commit(self, shape, k_all, v_all, prefix_len, an, na):
        kb = k_all.view(torch.int16).numpy().view(np.uint16)
        vb = v_all.view(torch.int16).numpy().view(np.uint16)
        oracle.kv_commit(kb, vb, prefix_len.numpy(), an.numpy(), na.numpy())


STEP_CFG = W.Config("T", 2, 5, 4, 2, 40, (1, 2, 2), 50, ("greedy", "mss"), 7, "test config (GQA 4/2)")


def _run_step(world, rank, kv_shard):
    import argparse
    import bench
    from paper_conf_asplos_miaoozcwzwzyssc24_b200 import step as S
    args = argparse.Namespace(layers=None, prefix=None, verify=None, batch=None, scaling="strong")
    cfg = STEP_CFG
    layout = S.make_layout(cfg.batch, world, rank, cfg.num_q_heads, cfg.num_kv_heads, kv_shard)
    wl = bench.Workload(cfg, args, layout, "cpu")
    shape_v = object() if kv_shard else None
    tree = (wl.tb.parent, wl.tb.depth, wl.tb.prefix_len, wl.tb.n_nodes)
    tree_v = (wl.tbv.parent, wl.tbv.depth, wl.tbv.prefix_len, wl.tbv.n_nodes) if kv_shard else tree
    shape = object()
    step = S.VerifyStep(OracleOps(), layout, shape, shape_v if kv_shard else shape, tree, tree_v, wl.verify,
                        wl.Dmax + 1, "cpu")
    out = torch.empty_like(wl.ai.q)
    step.prepare()
    for l in range(wl.L):
        step.attention(wl.ai.q[l], wl.ai.k_cache[l], wl.ai.v_cache[l], out[l], layer=l)
    inputs = {m: (wl.vi[m].logits, wl.vi[m].tree_tokens, wl.vi[m].draft_probs) for m in wl.verify}
    step.verify(inputs, seed=cfg.seed, offset=3)
    step.gather()
    step.commit(wl.ai.k_cache, wl.ai.v_cache)
    return (layout, step.accepted_all().numpy(), out.float().numpy(),
            wl.ai.k_cache.view(torch.int16).numpy().copy(), wl.tb.prefix_len.numpy().copy(), wl.tb.n_nodes.numpy())


def _step_worker(rank, world, port, kv_shard, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    torch.distributed.init_process_group("gloo", rank=rank, world_size=world)
    try:
        q.put((rank, _run_step(world, rank, kv_shard)))
    finally:
        torch.distributed.destroy_process_group()


@pytest.mark.parametrize("kv_shard", [False, True])
def test_step_plumbing_two_ranks_equals_one(kv_shard):
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_step_worker, args=(r, world, port, kv_shard, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = dict(q.get(timeout=300) for _ in range(world))
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    lay1, acc1, out1, k1, pl1, n1 = _run_step(1, 0, False)
    assert acc1[:, 0].min() >= 1                                   # every request accepted its root at least
    assert (acc1[:, 0] > 1).any()                                  # and some a longer path (rows really moved)
    for r in range(world):
        lay, acc, out, k, pl, n = res[r]
        np.testing.assert_array_equal(acc, acc1)                   # the gathered accepted rows, global order
        a = slice(lay.attn_lo, lay.attn_lo + lay.attn_cnt)
        np.testing.assert_array_equal(pl, pl1[a])                  # committed prefix lengths
        for i, b in enumerate(range(lay.attn_lo, lay.attn_lo + lay.attn_cnt)):
            P = pl1[b]
            np.testing.assert_array_equal(k[:, i, :, :P], k1[:, b, lay.kv0:lay.kv0 + lay.nkv, :P])
            np.testing.assert_array_equal(out[:, i, :n1[b]], out1[:, b, :n1[b], lay.q0:lay.q0 + lay.nq])
