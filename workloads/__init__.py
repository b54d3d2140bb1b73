"""Seeded synthetic workloads shared by the oracle tests, the GPU parity tests and bench.py.

This module holds the INPUT RECIPE only (shapes, value distributions, tree shapes); it holds
none of the verified method's arithmetic (no attention, no verification, no commit).  Both the
oracle side and the CUDA side receive the same bytes from here.

Recipe (DESIGN.md §"Inputs"):
* q, k, v ~ N(0, 1) rounded to bf16 (tree-slot K/V are independent draws); ``peaky`` multiplies
  q by 4 to stress the online-softmax rescaling.
* prefix_len = P for every request, or ragged: P_b = P - (37 b mod max(P/4, 1)).
* token trees: the paper's static expansion <k1..km> (L476-483, Fig. 3), linearised in DFS
  preorder (Fig. 2 "Linearization" L314, Fig. 4); or seeded random trees (config C5).
* LLM logits l_u = 3 z (z ~ N(0,1), fp32); draft distribution at node u q_u = softmax(l_u + tau e).
  Greedy trees take the top-k_i draft tokens of the parent (expansion method, L455-468);
  MSS trees draw each child i.i.d. from q_parent (reading R13) and draft_probs[c] = q_parent(c).
* Cache slots at or beyond P_b + n_b may be poisoned with NaN (tests) to prove they are unread.
"""
from __future__ import annotations

import dataclasses
import math
from typing import List, Optional, Sequence, Tuple

import numpy as np
import torch

HEAD_DIM = 128


# --------------------------------------------------------------------------------------------
# token-tree shapes
# --------------------------------------------------------------------------------------------

def expansion_tree(ks: Sequence[int]) -> Tuple[np.ndarray, np.ndarray]:
    """Tree of the static expansion config <k1, ..., km> (L476-483): step i expands every node
    at depth i-1 into k_i children.  Returned in DFS preorder as (parent, depth) int32 arrays;
    |N| = 1 + sum_i prod_{j<=i} k_j (Fig. 3: <2,2,1> -> 11 nodes)."""
    parent: List[int] = []
    depth: List[int] = []

    def visit(par: int, d: int) -> None:
        me = len(parent)
        parent.append(par)
        depth.append(d)
        if d < len(ks):
            for _ in range(ks[d]):
                visit(me, d + 1)

    visit(-1, 0)
    return np.asarray(parent, np.int32), np.asarray(depth, np.int32)


def random_tree(n: int, max_depth: int, max_fanout: int, rng: np.random.Generator
                ) -> Tuple[np.ndarray, np.ndarray]:
    """Seeded random token tree with exactly n nodes, depth <= max_depth, fanout <= max_fanout,
    returned in DFS preorder."""
    assert n >= 1
    children: List[List[int]] = [[]]
    depth = [0]
    while len(depth) < n:
        cands = [u for u in range(len(depth)) if depth[u] < max_depth and len(children[u]) < max_fanout]
        u = int(rng.choice(cands))
        children.append([])
        depth.append(depth[u] + 1)
        children[u].append(len(depth) - 1)
    # relabel in DFS preorder
    order: List[int] = []

    def dfs(u: int) -> None:
        order.append(u)
        for c in children[u]:
            dfs(c)

    dfs(0)
    new_id = {old: i for i, old in enumerate(order)}
    parent = np.full(n, -1, np.int32)
    dep = np.zeros(n, np.int32)
    for old in order:
        for c in children[old]:
            parent[new_id[c]] = new_id[old]
        dep[new_id[old]] = depth[old]
    return parent, dep


def chain_tree(n: int) -> Tuple[np.ndarray, np.ndarray]:
    return np.arange(-1, n - 1, dtype=np.int32), np.arange(n, dtype=np.int32)


# --------------------------------------------------------------------------------------------
# configs (BASELINE.json configs[0..4]; tree shapes resolved in SURVEY.md §8(c) A17)
# --------------------------------------------------------------------------------------------

@dataclasses.dataclass
class Config:
    name: str
    layers: int
    batch: int
    num_q_heads: int
    num_kv_heads: int
    prefix: int
    expansion: Optional[Tuple[int, ...]]
    vocab: int
    verify: Tuple[str, ...]
    seed: int
    description: str

    @property
    def tree(self) -> Tuple[np.ndarray, np.ndarray]:
        assert self.expansion is not None
        return expansion_tree(self.expansion)

    @property
    def n_nodes(self) -> int:
        return int(self.tree[0].shape[0])

    @property
    def max_depth(self) -> int:
        return len(self.expansion)


CONFIGS = {
    "C1": Config("C1", 1, 1, 32, 32, 128, (1, 2, 2, 2), 32000, ("greedy",), 1,
                 "1 request, single attention layer 32x128, prefix 128, 16-node tree <1,2,2,2>, greedy, V=32000"),
    "C2": Config("C2", 32, 16, 32, 32, 2048, (1, 1, 3, 1, 1, 1, 1, 1), 32000, ("greedy", "mss"), 2,
                 "LLaMA-7B shape: 32 layers x 32 heads x 128, bf16, batch 16, prefix 2048, tree <1,1,3,1,1,1,1,1> (21 nodes), greedy + MSS, V=32000"),
    "C3": Config("C3", 80, 32, 64, 8, 4096, (1, 2, 2, 2, 2, 2), 32000, ("greedy",), 3,
                 "LLaMA-2-70B shape GQA 64q/8kv x 128, 80 layers, batch 32, prefix 4096, 64-node tree <1,2,2,2,2,2>"),
    "C4": Config("C4", 48, 64, 56, 56, 1024, (8, 4, 1, 1, 1, 1, 1, 1), 50272, ("mss",), 4,
                 "OPT-30B shape 56 heads x 128, 48 layers, batch 64, prefix 1024, tree <8,4,1,1,1,1,1,1> (233 nodes), MSS, V=50272"),
}

# tau of the draft noise, calibrated once with the oracle so that the realised mean accepted
# length falls inside the paper's Table 2 range (greedy 2.18-3.91, stochastic 1.64-2.38 tokens
# per step, L1117-1127).  See DESIGN.md §"Inputs".
TAU_GREEDY = 1.0
TAU_MSS = 1.0
LOGIT_SCALE = 3.0


def ragged_prefix(P: int, B: int) -> np.ndarray:
    m = max(P // 4, 1)
    return np.asarray([P - (37 * b) % m for b in range(B)], np.int32)


def _gen(seed: int, device) -> torch.Generator:
    g = torch.Generator(device=device)
    g.manual_seed(int(seed))
    return g


def randn_bf16(shape, seed: int, device="cpu", scale: float = 1.0) -> torch.Tensor:
    x = torch.randn(tuple(shape), generator=_gen(seed, device), device=device, dtype=torch.float32)
    if scale != 1.0:
        x.mul_(scale)
    return x.to(torch.bfloat16)


# --------------------------------------------------------------------------------------------
# attention inputs
# --------------------------------------------------------------------------------------------

@dataclasses.dataclass
class TreeBatch:
    parent: torch.Tensor      # int32 [B][Nmax]
    depth: torch.Tensor       # int32 [B][Nmax]
    prefix_len: torch.Tensor  # int32 [B]
    n_nodes: torch.Tensor     # int32 [B]
    max_nodes: int
    max_depth: int


def make_tree_batch(trees: Sequence[Tuple[np.ndarray, np.ndarray]], prefix_len: Sequence[int],
                    max_nodes: Optional[int] = None, max_depth: Optional[int] = None,
                    device="cpu") -> TreeBatch:
    B = len(trees)
    Nmax = max_nodes or max(int(p.shape[0]) for p, _ in trees)
    parent = np.full((B, Nmax), -1, np.int32)
    depth = np.zeros((B, Nmax), np.int32)
    n = np.zeros(B, np.int32)
    for b, (p, d) in enumerate(trees):
        parent[b, :p.shape[0]] = p
        depth[b, :d.shape[0]] = d
        n[b] = p.shape[0]
    md = max_depth if max_depth is not None else int(depth.max())
    t = lambda a: torch.from_numpy(np.ascontiguousarray(a)).to(device)
    return TreeBatch(t(parent), t(depth), t(np.asarray(prefix_len, np.int32)), t(n), Nmax, md)


@dataclasses.dataclass
class AttnInputs:
    q: torch.Tensor        # bf16 [L][B][Nmax][Hq][D]
    k_cache: torch.Tensor  # bf16 [L][B][Hkv][Smax][D]
    v_cache: torch.Tensor
    tree: TreeBatch
    smax: int


def make_attention_inputs(tree: TreeBatch, layers: int, num_q_heads: int, num_kv_heads: int,
                          smax: int, seed: int, device="cpu", peaky: bool = False,
                          poison: bool = False, cache_layers: Optional[int] = None) -> AttnInputs:
    """q, K, V ~ N(0,1) -> bf16.  ``poison`` writes NaN into every slot >= P_b + n_b."""
    B, Nmax = tree.parent.shape
    D = HEAD_DIM
    L = layers
    q = torch.empty((L, B, Nmax, num_q_heads, D), dtype=torch.bfloat16, device=device)
    Lc = cache_layers if cache_layers is not None else L
    k = torch.empty((Lc, B, num_kv_heads, smax, D), dtype=torch.bfloat16, device=device)
    v = torch.empty_like(k)
    for l in range(L):
        q[l] = randn_bf16(q.shape[1:], 100 * seed + 1 + 1000 * l, device, 4.0 if peaky else 1.0)
    for l in range(Lc):
        k[l] = randn_bf16(k.shape[1:], 100 * seed + 2 + 1000 * l, device)
        v[l] = randn_bf16(v.shape[1:], 100 * seed + 3 + 1000 * l, device)
    if poison:
        pl = tree.prefix_len.cpu().numpy()
        nn_ = tree.n_nodes.cpu().numpy()
        for b in range(B):
            end = int(pl[b] + nn_[b])
            if end < smax:
                k[:, b, :, end:, :] = float("nan")
                v[:, b, :, end:, :] = float("nan")
    return AttnInputs(q, k, v, tree, smax)


# --------------------------------------------------------------------------------------------
# verification inputs
# --------------------------------------------------------------------------------------------

@dataclasses.dataclass
class VerifyInputs:
    logits: torch.Tensor       # fp32 [B][Nmax][V]
    draft_probs: torch.Tensor  # fp32 [B][Nmax][V]; row c = q_parent(c) (row 0 unused: zeros)
    tree_tokens: torch.Tensor  # int32 [B][Nmax]


def make_verify_inputs(tree: TreeBatch, vocab: int, seed: int, mode: str, device="cpu",
                       tau: Optional[float] = None, logit_scale: float = LOGIT_SCALE
                       ) -> VerifyInputs:
    """Synthetic LLM logits and SSM draft distributions; tree tokens drafted from them.

    mode "greedy": children of u are the top-k draft tokens of q_u (k = number of children);
    mode "mss":    children of u are i.i.d. draws from q_u.  The root token is arbitrary (0)."""
    B, Nmax = tree.parent.shape
    if tau is None:
        tau = TAU_GREEDY if mode == "greedy" else TAU_MSS
    g = _gen(100 * seed + 7, device)
    logits = torch.randn((B, Nmax, vocab), generator=g, device=device, dtype=torch.float32)
    logits.mul_(logit_scale)
    noise = torch.randn((B, Nmax, vocab), generator=g, device=device, dtype=torch.float32)
    q = torch.softmax(logits + tau * noise, dim=-1)
    del noise
    parent = tree.parent.cpu().numpy()
    n_nodes = tree.n_nodes.cpu().numpy()
    tokens = np.zeros((B, Nmax), np.int32)
    draft = torch.zeros((B, Nmax, vocab), dtype=torch.float32, device=device)
    gs = _gen(100 * seed + 8, device)
    for b in range(B):
        n = int(n_nodes[b])
        kids = {}
        for c in range(1, n):
            kids.setdefault(int(parent[b, c]), []).append(c)
        for u, cs in kids.items():
            if mode == "greedy":
                top = torch.topk(q[b, u], len(cs)).indices.cpu().numpy()
                toks = top
            else:
                toks = torch.multinomial(q[b, u], len(cs), replacement=True, generator=gs).cpu().numpy()
            for c, t in zip(cs, toks):
                tokens[b, c] = int(t)
                draft[b, c] = q[b, u]
    return VerifyInputs(logits, draft, torch.from_numpy(tokens).to(device))


def config_tree_batch(cfg: Config, device="cpu", ragged: bool = False,
                      batch: Optional[int] = None) -> TreeBatch:
    B = batch or cfg.batch
    p, d = cfg.tree
    pl = ragged_prefix(cfg.prefix, B) if ragged else np.full(B, cfg.prefix, np.int32)
    return make_tree_batch([(p, d)] * B, pl, device=device, max_depth=cfg.max_depth)


def c5_points():
    """Config C5: the sweep tree size x batch x prefix (one layer per point)."""
    pts = []
    for n in (8, 16, 32, 64, 128, 256):
        for B in (1, 8, 64):
            for P in (512, 2048, 8192):
                pts.append((n, B, P))
    return pts


def random_tree_batch(B: int, n: int, P: int, seed: int, max_depth: int = 8, max_fanout: int = 8,
                      device="cpu", ragged_n: bool = False) -> TreeBatch:
    rng = np.random.default_rng(seed)
    trees = []
    for b in range(B):
        nb = n if not ragged_n else int(rng.integers(1, n + 1))
        # depth <= 8 with fanout <= 8 can hold at most 1 + 8 + ... nodes; clamp fanout need
        trees.append(random_tree(nb, max_depth, max_fanout, rng))
    return make_tree_batch(trees, [P] * B, max_nodes=n, max_depth=max_depth, device=device)


# --------------------------------------------------------------------------------------------
# per-request generation (multi-GPU bench): every request's tensors come from their own seeded
# generator, so a rank can materialise exactly its share of a GLOBAL problem (request range and /
# or kv-head range) and the values equal the N = 1 run's bit for bit (strong scaling)
# --------------------------------------------------------------------------------------------

def request_seed(seed: int, tensor_id: int, layer: int, rid: int) -> int:
    ss = np.random.SeedSequence([int(seed), int(tensor_id), int(layer), int(rid)])
    return int(ss.generate_state(1, np.uint64)[0] & np.uint64(2**63 - 1))


def make_request_attention_inputs(tree: TreeBatch, request_ids: Sequence[int], layers: int, num_q_heads: int,
                                  num_kv_heads: int, smax: int, seed: int, q_heads: Tuple[int, int] = None,
                                  kv_heads: Tuple[int, int] = None, device="cpu") -> AttnInputs:
    """q, K, V ~ N(0,1) -> bf16 for the global requests ``request_ids`` (rows of ``tree`` in the same
    order), keeping q-heads [q0, q0 + nq) and kv-heads [kv0, kv0 + nkv) of the global head counts."""
    B, Nmax = tree.parent.shape
    assert len(request_ids) == B
    q0, nq = q_heads or (0, num_q_heads)
    kv0, nkv = kv_heads or (0, num_kv_heads)
    D = HEAD_DIM
    q = torch.empty((layers, B, Nmax, nq, D), dtype=torch.bfloat16, device=device)
    k = torch.empty((layers, B, nkv, smax, D), dtype=torch.bfloat16, device=device)
    v = torch.empty_like(k)
    for l in range(layers):
        for i, rid in enumerate(request_ids):
            q[l, i] = randn_bf16((Nmax, num_q_heads, D), request_seed(seed, 1, l, rid), device)[:, q0:q0 + nq]
            k[l, i] = randn_bf16((num_kv_heads, smax, D), request_seed(seed, 2, l, rid), device)[kv0:kv0 + nkv]
            v[l, i] = randn_bf16((num_kv_heads, smax, D), request_seed(seed, 3, l, rid), device)[kv0:kv0 + nkv]
    return AttnInputs(q, k, v, tree, smax)


def make_request_verify_inputs(tree: TreeBatch, request_ids: Sequence[int], vocab: int, seed: int, mode: str,
                               device="cpu", tau: Optional[float] = None,
                               logit_scale: float = LOGIT_SCALE) -> VerifyInputs:
    """make_verify_inputs with one generator per global request (same recipe).  The LLM logits and the
    SSM distributions of a request do not depend on `mode`; only the drafting policy does (greedy:
    top-k children, MSS: i.i.d. draws), so both verifiers of a config see the same model outputs."""
    B, Nmax = tree.parent.shape
    if tau is None:
        tau = TAU_GREEDY if mode == "greedy" else TAU_MSS
    parent = tree.parent.cpu().numpy()
    n_nodes = tree.n_nodes.cpu().numpy()
    logits = torch.empty((B, Nmax, vocab), dtype=torch.float32, device=device)
    draft = torch.zeros((B, Nmax, vocab), dtype=torch.float32, device=device)
    tokens = np.zeros((B, Nmax), np.int32)
    for i, rid in enumerate(request_ids):
        g = _gen(request_seed(seed, 7, 0, rid), device)
        lg = torch.randn((Nmax, vocab), generator=g, device=device, dtype=torch.float32).mul_(logit_scale)
        noise = torch.randn((Nmax, vocab), generator=g, device=device, dtype=torch.float32)
        q = torch.softmax(lg + tau * noise, dim=-1)
        logits[i] = lg
        gs = _gen(request_seed(seed, 8, 0, rid), device)
        kids = {}
        for c in range(1, int(n_nodes[i])):
            kids.setdefault(int(parent[i, c]), []).append(c)
        for u, cs in kids.items():
            if mode == "greedy":
                toks = torch.topk(q[u], len(cs)).indices.cpu().numpy()
            else:
                toks = torch.multinomial(q[u], len(cs), replacement=True, generator=gs).cpu().numpy()
            for c, t in zip(cs, toks):
                tokens[i, c] = int(t)
                draft[i, c] = q[u]
    return VerifyInputs(logits, draft, torch.from_numpy(tokens).to(device))
