"""Multi-GPU plumbing of the verification step.

The hot path partitions by request: every (request, kv-head) is independent for tree attention and
KV commit, every request for verification.  Two layouts:
  * request sharding (C2, C4, C5): ranks own disjoint request ranges end to end;
  * kv-head sharding (GQA, C3): ranks own disjoint kv-head ranges (and their q-head groups) of every
    request for attention and KV commit, while verification stays request-sharded (the logits are
    per request); the gathered accepted paths let every rank commit its head shard of all requests.
Either way the only exchange is the tokens-only gather after verification (the
request manager and GPU workers "only communicate tokens").  MSS counters use global request ids, so
results are identical at any world size.  NCCL (over NVLink/NVSwitch) on GPUs; gloo for the CPU tests.
"""
from __future__ import annotations

from typing import Tuple

import torch


def shard_requests(batch_global: int, world: int, rank: int) -> Tuple[int, int]:
    """Contiguous request range [start, start + count) of `rank` (strong scaling split)."""
    base, rem = divmod(batch_global, world)
    start = rank * base + min(rank, rem)
    return start, base + (1 if rank < rem else 0)


def shard_kv_heads(num_q_heads: int, num_kv_heads: int, world: int, rank: int) -> Tuple[int, int, int, int]:
    """kv-head sharding: rank's kv-heads [kv0, kv0 + nkv) and their q-heads [q0, q0 + nq) (each
    kv-head keeps its whole GQA group, so attention needs no exchange).  Requires Hkv % world == 0."""
    if num_kv_heads % world != 0 or num_q_heads % num_kv_heads != 0:
        raise ValueError(f"cannot shard {num_kv_heads} kv-heads over {world} ranks")
    G = num_q_heads // num_kv_heads
    nkv = num_kv_heads // world
    kv0 = rank * nkv
    return kv0, nkv, kv0 * G, nkv * G


def global_request_ids(start: int, count: int, device) -> torch.Tensor:
    return torch.arange(start, start + count, dtype=torch.int32, device=device)


def pack_accepted(n_accepted: torch.Tensor, accepted_tokens: torch.Tensor,
                  accepted_nodes: torch.Tensor) -> torch.Tensor:
    """int32 [B][2 Lp + 1] = [n | tokens | nodes] (one contiguous row per request)."""
    B, Lp = accepted_tokens.shape
    out = torch.empty((B, 2 * Lp + 1), dtype=torch.int32, device=accepted_tokens.device)
    out[:, 0] = n_accepted
    out[:, 1:1 + Lp] = accepted_tokens
    out[:, 1 + Lp:] = accepted_nodes
    return out


def unpack_accepted(buf: torch.Tensor):
    Lp = (buf.shape[1] - 1) // 2
    return buf[:, 0], buf[:, 1:1 + Lp], buf[:, 1 + Lp:]


def gather_accepted(packed: torch.Tensor, out: torch.Tensor = None) -> torch.Tensor:
    """All-gather the per-rank packed rows (EQUAL row counts per rank) into [world·rows][2Lp+1].
    Uneven request shards go through `GatherPlan` (padding rows with n = 0)."""
    world = torch.distributed.get_world_size()
    if out is None:
        out = torch.empty((world * packed.shape[0], packed.shape[1]), dtype=packed.dtype, device=packed.device)
    if out.shape[0] != world * packed.shape[0]:
        raise ValueError(f"gather_accepted: out has {out.shape[0]} rows, expected {world} x {packed.shape[0]}")
    if torch.distributed.get_backend() == "nccl":
        torch.distributed.all_gather_into_tensor(out, packed)
    else:
        parts = list(out.chunk(world, dim=0))
        torch.distributed.all_gather(parts, packed)
        if parts[0].data_ptr() != out.data_ptr():
            out.copy_(torch.cat(parts, 0))
    return out


class GatherPlan:
    """The tokens-only exchange (a7) for `batch_global` requests split by `shard_requests` over
    `world` ranks: every rank contributes ceil(B / world) rows (its requests, then padding rows with
    n = 0, which every consumer treats as 'nothing accepted'), one all-gather, and `rows_of_all`
    gives the global requests in order (padding dropped)."""

    def __init__(self, batch_global: int, world: int, path_len: int, device):
        self.world, self.B, self.Lp = world, batch_global, path_len
        self.pad = -(-batch_global // world)
        self.counts = [shard_requests(batch_global, world, r)[1] for r in range(world)]
        idx = [r * self.pad + i for r in range(world) for i in range(self.counts[r])]
        self.index = torch.tensor(idx, dtype=torch.long, device=device)
        self.send = torch.zeros((self.pad, 2 * path_len + 1), dtype=torch.int32, device=device)
        self.recv = torch.zeros((world * self.pad, 2 * path_len + 1), dtype=torch.int32, device=device)

    def pack(self, n_accepted, accepted_tokens, accepted_nodes):
        cnt = n_accepted.shape[0]
        self.send[:cnt, 0] = n_accepted
        self.send[:cnt, 1:1 + self.Lp] = accepted_tokens
        self.send[:cnt, 1 + self.Lp:] = accepted_nodes
        return self.send

    def exchange(self):
        if self.world > 1:
            gather_accepted(self.send, self.recv)
        else:
            self.recv.copy_(self.send)
        return self.recv

    def rows_of_all(self) -> torch.Tensor:
        """[batch_global][2Lp+1] packed rows of every request in global order."""
        return self.recv.index_select(0, self.index)


class P2PGather:
    """NEXT-4a: one rank's buffers for the verifier-fused gather (include/specinfer.h,
    specinfer_gather_t) and the peer mappings of every other rank's buffers (CUDA IPC: over
    NVLink / NVSwitch between GPUs, plain device memory between processes on one GPU).

    `exchange(obj) -> [obj of rank 0, ..., obj of rank world-1]` shares picklable objects between the
    ranks (torch.distributed.all_gather_object, or queues in a test).  The row layout is GatherPlan's:
    request b of rank r at row r * pad + b, so GatherPlan.index selects the global requests."""

    def __init__(self, batch_global: int, world: int, rank: int, path_len: int, device, exchange=None):
        from torch.multiprocessing.reductions import reduce_tensor
        import paper_conf_asplos_miaoozcwzwzyssc24_b200 as spi
        if world > spi.MAX_PEERS:
            raise ValueError(f"P2PGather: at most {spi.MAX_PEERS} ranks")
        self.world, self.rank, self.B = world, rank, batch_global
        self.pad = -(-batch_global // world)
        self.row_len = 2 * path_len + 1
        i32 = dict(dtype=torch.int32, device=device)
        self.recv = torch.zeros((2, world * self.pad, self.row_len), **i32)
        self.flags = torch.zeros((world,), **i32)
        self.state = torch.zeros((2,), **i32)
        self.table = torch.zeros((world * self.pad, self.row_len), **i32)
        if world > 1:
            objs = exchange((reduce_tensor(self.recv), reduce_tensor(self.flags)))
            self.peers = []
            for r, ((f1, a1), (f2, a2)) in enumerate(objs):
                self.peers.append((self.recv, self.flags) if r == rank else (f1(*a1), f2(*a2)))
        else:
            self.peers = [(self.recv, self.flags)]
        d = spi.GatherDesc()
        d.world, d.rank, d.rows_per_rank, d.row_len = world, rank, self.pad, self.row_len
        for r, (rv, fl) in enumerate(self.peers):
            d.recv[r] = rv.data_ptr()
            d.flags[r] = fl.data_ptr()
        d.state = self.state.data_ptr()
        self.desc = d
        self.spi = spi

    def wait(self):
        """Device-side wait for this step's rows of every rank; returns the table (global order via
        GatherPlan.index)."""
        self.spi.specinfer_gather_wait(self.desc, self.table)
        return self.table


def all_gather_object_exchange(obj):
    out = [None] * torch.distributed.get_world_size()
    torch.distributed.all_gather_object(out, obj)
    return out
