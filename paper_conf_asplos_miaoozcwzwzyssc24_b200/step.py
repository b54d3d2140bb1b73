"""One verification iteration of the hot path for one rank (a0 -> L x (a1-a3) ->
a4 | a5 -> a7 -> a6), in either multi-GPU layout of dist.py, as stream-ordered segments that the
bench captures as CUDA graphs.

    layout = make_layout(batch_global, world, rank, Hq, Hkv, kv_shard)
    step = VerifyStep(DeviceOps(), layout, shapes, trees, modes, path_len, device)
    step.prepare(); for l: step.attention(q[l], k[l], v[l], out[l], layer=l)
    step.verify(inputs, seed, offset); step.gather(); step.commit(k_all, v_all)

The device work is the library through `ops` (DeviceOps = the C ABI of libspecinfer.so; there is no
other implementation in this package).  The object only routes buffers between the calls: which
requests and heads this rank owns, the tokens-only gather and which accepted
paths the commit consumes.  tests/test_multirank.py drives the same object with a host stand-in for
`ops` under gloo to check that the plumbing gives N = 1's results bit for bit.
"""
from __future__ import annotations

import dataclasses
from typing import Optional, Sequence, Tuple

import torch

from . import dist as D


@dataclasses.dataclass
class Layout:
    """What rank `rank` of `world` owns.

    request sharding: verification AND attention / commit over requests [req_lo, req_lo + req_cnt)
    with every head.  kv-head sharding (GQA): attention / commit over ALL requests for kv-heads
    [kv0, kv0 + nkv) and their q-heads [q0, q0 + nq); verification over [req_lo, req_lo + req_cnt)."""
    world: int
    rank: int
    kv_shard: bool
    batch_global: int
    req_lo: int
    req_cnt: int
    attn_lo: int
    attn_cnt: int
    q0: int
    nq: int
    kv0: int
    nkv: int

    @property
    def verify_ids(self) -> range:
        return range(self.req_lo, self.req_lo + self.req_cnt)

    @property
    def attn_ids(self) -> range:
        return range(self.attn_lo, self.attn_lo + self.attn_cnt)


def make_layout(batch_global: int, world: int, rank: int, num_q_heads: int, num_kv_heads: int,
                kv_shard: bool) -> Layout:
    lo, cnt = D.shard_requests(batch_global, world, rank)
    if kv_shard:
        kv0, nkv, q0, nq = D.shard_kv_heads(num_q_heads, num_kv_heads, world, rank)
        return Layout(world, rank, True, batch_global, lo, cnt, 0, batch_global, q0, nq, kv0, nkv)
    return Layout(world, rank, False, batch_global, lo, cnt, lo, cnt, 0, num_q_heads, 0, num_kv_heads)


class DeviceOps:
    """The library calls the step is made of (argument marshalling in __init__.py)."""

    concurrent_verifiers = True   # independent verifiers may run on a side stream (own workspace regions)

    def __init__(self):
        import paper_conf_asplos_miaoozcwzwzyssc24_b200 as spi   # the binding (no CPU path)
        self.spi = spi

    def state(self, shape, parent, depth, prefix_len, n_nodes):
        return self.spi.TreeState.create(shape, parent, depth, prefix_len, n_nodes)

    def prepare(self, st):
        st.prepare()

    def attention(self, st, q, k, v, out, prefetch: bool):
        st.attention(q, k, v, out, prefetch=prefetch)

    def verify_greedy(self, shape, st, logits, tokens, parent, n_nodes, an, at, na, gather=None):
        self.spi.specinfer_verify_greedy(shape, logits, tokens, parent, n_nodes, an, at, na, st.workspace,
                                         gather=gather)

    def verify_mss(self, shape, st, logits, tokens, parent, n_nodes, draft, temperature, seed, offset, rids, an, at,
                   na, gather=None):
        self.spi.specinfer_verify_mss(shape, logits, tokens, parent, n_nodes, draft, temperature, seed, offset, rids,
                                      an, at, na, st.workspace, gather=gather)

    def kv_commit(self, shape, k_all, v_all, prefix_len, an, na):
        self.spi.specinfer_kv_commit(shape, k_all, v_all, prefix_len, an, na)


class VerifyStep:
    """Buffers and routing of one rank's iteration.  `attn_tree` / `verify_tree` are
    (parent, depth, prefix_len, n_nodes) of the attention batch (layout.attn_ids) and of the
    verification batch (layout.verify_ids); with request sharding they are the same tensors."""

    def __init__(self, ops, layout: Layout, shape_attn, shape_verify, attn_tree: Tuple, verify_tree: Tuple,
                 modes: Sequence[str], path_len: int, device, commit_mode: Optional[str] = None,
                 p2p: Optional["D.P2PGather"] = None):
        """p2p: NEXT-4a, the committed verifier publishes its rows to every rank itself (peer stores +
        flags) and gather() is a device-side wait; None: the NCCL / gloo all-gather (GatherPlan)."""
        self.ops, self.layout = ops, layout
        self.shape_attn, self.shape_verify = shape_attn, shape_verify
        self.attn_tree, self.verify_tree = attn_tree, verify_tree
        self.modes = tuple(modes)
        self.commit_mode = commit_mode or ("greedy" if "greedy" in self.modes else "mss")
        assert self.commit_mode in self.modes
        self.Lp = path_len
        self.st = ops.state(shape_attn, *attn_tree)
        same = (not layout.kv_shard) and shape_verify is shape_attn
        self.st_v = self.st if same else ops.state(shape_verify, *verify_tree)
        B = layout.req_cnt
        i32 = dict(dtype=torch.int32, device=device)
        self.res = {m: (torch.full((B, path_len), -1, **i32), torch.full((B, path_len), -1, **i32),
                        torch.zeros((B,), **i32)) for m in self.modes}   # (nodes, tokens, n) per verifier
        self.rids = torch.arange(layout.req_lo, layout.req_lo + B, **i32)
        self.plan = D.GatherPlan(layout.batch_global, layout.world, path_len, device)
        self.p2p = p2p
        self.an_all = torch.zeros((layout.batch_global, path_len), **i32)
        self.device, self._side, self._pending = device, None, False
        self.na_all = torch.zeros((layout.batch_global,), **i32)
        self._layer = 0

    # ---- a0 ----
    def prepare(self):
        self.ops.prepare(self.st)
        if self.st_v is not self.st:
            self.ops.prepare(self.st_v)
        self._layer = 0

    # ---- a1-a3, one layer ----
    def attention(self, q, k, v, out, layer: Optional[int] = None):
        # layers after the first may stage committed-prefix tiles before the previous launch ends
        # (nothing between two attention launches writes the prefix or the schedule)
        first = (layer == 0) if layer is not None else (self._layer == 0)
        self.ops.attention(self.st, q, k, v, out, prefetch=not first)
        self._layer += 1

    # ---- a4 | a5 ----
    def verify(self, inputs: dict, seed: int, offset: int = 0, temperature: float = 1.0, join: bool = True):
        """inputs[mode] = (logits, tree_tokens, draft_probs or None) for this rank's requests.  With more than
        one verifier, the ones whose result is not committed run on a side stream, concurrently with the
        committed one (they use separate workspace counters / buffers); the caller's stream joins them now,
        or, with join=False, at join() -- so that gather / commit (which need only the committed verifier)
        overlap them too."""
        parent, _, _, n_nodes = self.verify_tree

        def one(m):
            an, at, na = self.res[m]
            logits, tokens, draft = inputs[m]
            kw = {"gather": self.p2p.desc} if (self.p2p is not None and m == self.commit_mode) else {}
            if m == "greedy":
                self.ops.verify_greedy(self.shape_verify, self.st_v, logits, tokens, parent, n_nodes, an, at, na, **kw)
            else:
                self.ops.verify_mss(self.shape_verify, self.st_v, logits, tokens, parent, n_nodes, draft,
                                    temperature, seed, offset, self.rids, an, at, na, **kw)

        others = [m for m in self.modes if m != self.commit_mode]
        if others and getattr(self.ops, "concurrent_verifiers", False):
            main = torch.cuda.current_stream(self.device)
            if self._side is None:
                self._side = torch.cuda.Stream(self.device)
            self._side.wait_stream(main)
            with torch.cuda.stream(self._side):
                for m in others:
                    one(m)
            one(self.commit_mode)
            self._pending = True
            if join:
                self.join()
        else:
            for m in self.modes:
                one(m)

    def join(self):
        """The caller's stream waits for the verifiers still running on the side stream."""
        if self._pending:
            torch.cuda.current_stream(self.device).wait_stream(self._side)
            self._pending = False

    # ---- a7 ----
    def gather(self):
        """Tokens-only all-gather of the committed verifier's rows (n | tokens | nodes); at N = 1 a
        copy, so the kv-sharded path is exercised on one GPU too."""
        if self.p2p is not None:
            table = self.p2p.wait()          # the verifier already stored the rows on every rank
        else:
            an, at, na = self.res[self.commit_mode]
            self.plan.pack(na, at, an)
            table = self.plan.exchange()
        if self.layout.kv_shard:
            rows = table.index_select(0, self.plan.index)
            n_all, _, nodes_all = D.unpack_accepted(rows)
            self.na_all.copy_(n_all)
            self.an_all.copy_(nodes_all)
        return table

    # ---- a6 ----
    def commit(self, k_all, v_all):
        prefix_len = self.attn_tree[2]
        if self.layout.kv_shard:
            src = (self.an_all, self.na_all)     # every request's path -> this rank's head shard
        else:
            an, _, na = self.res[self.commit_mode]
            src = (an, na)
        self.ops.kv_commit(self.shape_attn, k_all, v_all, prefix_len, *src)

    def accepted(self, mode: Optional[str] = None):
        """(n_accepted, accepted_tokens, accepted_nodes) of this rank's requests."""
        an, at, na = self.res[mode or self.commit_mode]
        return na, at, an

    def accepted_all(self) -> torch.Tensor:
        """Packed rows of every global request after gather() (global order)."""
        table = self.p2p.table if self.p2p is not None else self.plan.recv
        return table.index_select(0, self.plan.index)
