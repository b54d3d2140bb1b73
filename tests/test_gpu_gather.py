"""NEXT-4a: the tokens-only gather fused into the verifiers (include/specinfer.h
specinfer_verify_*_ex / specinfer_gather_wait).  The verifier's last CTA of every request stores the
packed row [n | tokens | nodes] into every rank's receive table and the rank's last request releases
an epoch flag on every rank; gather_wait acquires all flags.

Checked here on the one GPU of the test box:
  * world 1 (the rank publishes to itself), eager and inside a replayed CUDA graph, several steps
    (epoch parity): the table equals the packed outputs of the plain verifier;
  * world 2 as two processes on the same GPU sharing their tables and flags through CUDA IPC (the
    mapping the bench uses between GPUs), an uneven request split (7 requests = 4 + 3), three steps
    with different MSS offsets: every rank's gathered table equals the packed rows of the
    single-process verifier over the whole batch (global request ids), i.e. what the NCCL all-gather
    (GatherPlan) delivers.
"""
import os

import numpy as np
import pytest
import torch
import torch.multiprocessing as mp

import workloads as W
from paper_conf_asplos_miaoozcwzwzyssc24_b200 import dist as D

pytestmark = pytest.mark.gpu

if torch.cuda.is_available():
    import paper_conf_asplos_miaoozcwzwzyssc24_b200 as spi

DEV = "cuda:0"
B_GLOBAL, V, NMAX, DMAX = 7, 300, 24, 6
LP = DMAX + 1


def _problem(device):
    rng = np.random.default_rng(17)
    trees = [W.random_tree(int(rng.integers(1, NMAX + 1)), DMAX, 4, rng) for _ in range(B_GLOBAL)]
    tb = W.make_tree_batch(trees, [5] * B_GLOBAL, max_nodes=NMAX, max_depth=DMAX, device=device)
    vi = W.make_verify_inputs(tb, V, seed=8, mode="mss", device=device)
    return tb, vi


def _slice_tb(tb, lo, cnt):
    s = slice(lo, lo + cnt)
    return W.TreeBatch(tb.parent[s].contiguous(), tb.depth[s].contiguous(), tb.prefix_len[s].contiguous(),
                       tb.n_nodes[s].contiguous(), tb.max_nodes, tb.max_depth)


def _verify(tb, vi, lo, cnt, offset, gather=None, mode="mss"):
    t = _slice_tb(tb, lo, cnt)
    shape = spi.make_shape(cnt, NMAX, 1, 1, NMAX + 8, vocab=V, max_depth=DMAX)
    st = spi.TreeState.create(shape, t.parent, t.depth, t.prefix_len, t.n_nodes)
    st.prepare()
    an = torch.empty((cnt, LP), dtype=torch.int32, device=DEV)
    at, na = torch.empty_like(an), torch.empty((cnt,), dtype=torch.int32, device=DEV)
    s = slice(lo, lo + cnt)
    if mode == "mss":
        rids = torch.arange(lo, lo + cnt, dtype=torch.int32, device=DEV)
        spi.specinfer_verify_mss(shape, vi.logits[s].contiguous(), vi.tree_tokens[s].contiguous(), t.parent,
                                 t.n_nodes, vi.draft_probs[s].contiguous(), 1.0, 3, offset, rids, an, at, na,
                                 st.workspace, gather=gather)
    else:
        spi.specinfer_verify_greedy(shape, vi.logits[s].contiguous(), vi.tree_tokens[s].contiguous(), t.parent,
                                    t.n_nodes, an, at, na, st.workspace, gather=gather)
    return na, at, an


def _expected(offset, mode="mss"):
    tb, vi = _problem(DEV)
    na, at, an = _verify(tb, vi, 0, B_GLOBAL, offset, mode=mode)
    torch.cuda.synchronize()
    return D.pack_accepted(na, at, an).cpu().numpy()


@pytest.mark.parametrize("mode", ["greedy", "mss"])
def test_fused_gather_world1_eager_and_graph(mode):
    tb, vi = _problem(DEV)
    g = D.P2PGather(B_GLOBAL, 1, 0, LP, DEV)
    plan = D.GatherPlan(B_GLOBAL, 1, LP, DEV)
    for step in range(3):   # epochs 1..3, both table buffers
        na, at, an = _verify(tb, vi, 0, B_GLOBAL, step, gather=g.desc, mode=mode)
        table = g.wait()
        torch.cuda.synchronize()
        np.testing.assert_array_equal(table.index_select(0, plan.index).cpu().numpy(),
                                      D.pack_accepted(na, at, an).cpu().numpy())
        assert int(g.state[0]) == step + 1 and int(g.state[1]) == 0
    # inside a CUDA graph: the epoch lives in device memory, so replays keep synchronising
    t = _slice_tb(tb, 0, B_GLOBAL)
    shape = spi.make_shape(B_GLOBAL, NMAX, 1, 1, NMAX + 8, vocab=V, max_depth=DMAX)
    st = spi.TreeState.create(shape, t.parent, t.depth, t.prefix_len, t.n_nodes)
    an = torch.empty((B_GLOBAL, LP), dtype=torch.int32, device=DEV)
    at, na = torch.empty_like(an), torch.empty((B_GLOBAL,), dtype=torch.int32, device=DEV)
    s = torch.cuda.Stream()
    s.wait_stream(torch.cuda.current_stream())
    with torch.cuda.stream(s):
        st.prepare()
    torch.cuda.synchronize()
    graph = torch.cuda.CUDAGraph()
    with torch.cuda.graph(graph, stream=s):
        if mode == "mss":
            rids = torch.arange(0, B_GLOBAL, dtype=torch.int32, device=DEV)
            spi.specinfer_verify_mss(shape, vi.logits, vi.tree_tokens, t.parent, t.n_nodes, vi.draft_probs, 1.0, 3,
                                     0, rids, an, at, na, st.workspace, gather=g.desc)
        else:
            spi.specinfer_verify_greedy(shape, vi.logits, vi.tree_tokens, t.parent, t.n_nodes, an, at, na,
                                        st.workspace, gather=g.desc)
        g.wait()
    exp = _expected(0, mode)
    for rep in range(3):
        g.table.zero_()
        graph.replay()
        torch.cuda.synchronize()
        np.testing.assert_array_equal(g.table.index_select(0, plan.index).cpu().numpy(), exp)
        assert int(g.state[0]) == 4 + rep


def _rank_proc(rank, world, q_out, q_in, q_res):
    torch.cuda.set_device(0)
    tb, vi = _problem(DEV)
    lo, cnt = D.shard_requests(B_GLOBAL, world, rank)

    def exchange(obj):
        q_out.put((rank, obj))
        return q_in.get(timeout=120)

    g = D.P2PGather(B_GLOBAL, world, rank, LP, DEV, exchange=exchange)
    plan = D.GatherPlan(B_GLOBAL, world, LP, DEV)
    tables = []
    for step in range(3):
        _verify(tb, vi, lo, cnt, offset=step, gather=g.desc)
        table = g.wait()
        torch.cuda.synchronize()
        tables.append(table.index_select(0, plan.index).cpu().numpy())
    q_res.put((rank, tables))
    q_in.get(timeout=120)   # keep the IPC-shared buffers alive until every rank is done


def test_fused_gather_two_processes_ipc():
    world = 2
    ctx = mp.get_context("spawn")
    q_out, q_res = ctx.Queue(), ctx.Queue()
    q_in = [ctx.Queue() for _ in range(world)]
    procs = [ctx.Process(target=_rank_proc, args=(r, world, q_out, q_in[r], q_res)) for r in range(world)]
    for p in procs:
        p.start()
    objs = dict(q_out.get(timeout=300) for _ in range(world))
    for r in range(world):
        q_in[r].put([objs[i] for i in range(world)])
    res = dict(q_res.get(timeout=300) for _ in range(world))
    for r in range(world):
        q_in[r].put("done")
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    for step in range(3):
        exp = _expected(step)
        for r in range(world):
            np.testing.assert_array_equal(res[r][step], exp)
