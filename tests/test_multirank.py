"""World-size-2 gloo test of the multi-GPU host logic (request sharding, global request ids, the
tokens-only all-gather).  The per-rank "device" work is the oracle, so this runs on CPU; the
invariant checked is that the gathered results equal a single-process run on the whole batch
(integer outputs bit-identical across world sizes)."""
import os
import socket

import numpy as np
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
