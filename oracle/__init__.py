"""CPU oracle for SpecInfer's token-tree verification hot path — TEST INFRASTRUCTURE ONLY.

Plain fp64 C (``specinfer_oracle.c``) behind ctypes, operating on numpy host arrays.
Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py`` (its ``cpu_baseline`` leg and
``--impl reference``) may import this package.  The product path
(``paper_conf_asplos_miaoozcwzwzyssc24_b200``) never imports it; the two share no code.

Each wrapper cites the PAPER.md passage its C function follows (see the C file header).
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "specinfer_oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")

_lib = None


def build(force: bool = False) -> str:
    """Compile the oracle with gcc (-O2 -fopenmp, fp64, no fast-math)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-fopenmp", "-fPIC", "-shared", "-std=c11",
                               "-Wall", "-o", tmp, _SRC, "-lm"])
        os.replace(tmp, _LIB)
    return _LIB


def lib():
    global _lib
    if _lib is None:
        _lib = ctypes.CDLL(build())
        i32, i64, u64, dbl, vp = (ctypes.c_int32, ctypes.c_int64, ctypes.c_uint64,
                                  ctypes.c_double, ctypes.c_void_p)
        _lib.oracle_validate_tree.argtypes = [i32, i32, i32, vp, vp, i32, i32]
        _lib.oracle_validate_tree.restype = ctypes.c_int
        _lib.oracle_tree_attention.argtypes = [i32, i32, i32, i32, i32, i32, i32, dbl,
                                               vp, vp, vp, vp, vp, vp, vp, vp]
        _lib.oracle_kv_commit.argtypes = [i32, i32, i32, i32, i32, i64, i32, vp, vp, vp, vp, vp]
        _lib.oracle_verify_greedy.argtypes = [i32, i32, i32, i32, i32, i32, vp, vp, vp, vp, vp,
                                              vp, vp, vp, vp]
        _lib.oracle_verify_mss.argtypes = [i32, i32, i32, i32, i32, i32, vp, vp, vp, vp, vp, vp,
                                           vp, dbl, u64, u64, vp, vp, vp, vp, vp,
                                           i32, vp, vp, vp, vp, vp]
        _lib.oracle_verify_ns.argtypes = [i32, i32, i32, i32, i32, i32, vp, vp, vp, vp, vp, vp,
                                          dbl, u64, u64, vp, vp, vp, vp, vp,
                                          i32, vp, vp, vp, vp, vp]
        _lib.oracle_philox4x32_10.argtypes = [vp, vp, vp]
        _lib.oracle_set_num_threads.argtypes = [i32]
        _lib.oracle_set_num_threads.restype = None
    return _lib


def set_num_threads(n: int) -> None:
    """OpenMP threads of the oracle's loops (timing only; results do not depend on it)."""
    lib().oracle_set_num_threads(int(n))


def _p(a):
    return None if a is None else a.ctypes.data_as(ctypes.c_void_p)


def _c(a, dtype):
    return np.ascontiguousarray(a, dtype=dtype)


def bf16_bits(x) -> np.ndarray:
    """View a bf16 array (numpy uint16 bits or torch bf16 tensor on CPU) as uint16 bits."""
    if hasattr(x, "view") and hasattr(x, "dtype") and str(x.dtype) == "torch.bfloat16":
        import torch
        return x.contiguous().view(torch.int16).numpy().view(np.uint16)
    return _c(x, np.uint16)


def validate_tree(parent, depth, prefix_len, n_nodes, nmax, max_depth, smax) -> int:
    parent = _c(parent, np.int32)
    depth = None if depth is None else _c(depth, np.int32)
    return lib().oracle_validate_tree(nmax, max_depth, smax, _p(parent), _p(depth),
                                      int(prefix_len), int(n_nodes))


def tree_attention(q, k, v, parent, depth, prefix_len, n_nodes, *, max_depth=255,
                   sm_scale=None, out=None) -> np.ndarray:
    """c1 (Def. 4.1).  q [B][Nmax][Hq][D], k/v [B][Hkv][Smax][D] as bf16
    bits (uint16); returns fp64 out [B][Nmax][Hq][D] (rows i >= n_nodes[b] are NaN)."""
    q, k, v = bf16_bits(q), bf16_bits(k), bf16_bits(v)
    B, Nmax, Hq, D = q.shape
    _, Hkv, Smax, _ = k.shape
    assert k.shape == v.shape and k.shape[0] == B and k.shape[3] == D and Hq % Hkv == 0
    if sm_scale is None:
        sm_scale = 1.0 / np.sqrt(D)
    parent = _c(parent, np.int32).reshape(B, Nmax)
    depth = None if depth is None else _c(depth, np.int32).reshape(B, Nmax)
    prefix_len, n_nodes = _c(prefix_len, np.int32), _c(n_nodes, np.int32)
    if out is None:
        out = np.full((B, Nmax, Hq, D), np.nan, dtype=np.float64)
    lib().oracle_tree_attention(B, Nmax, Hq, Hkv, D, Smax, max_depth, float(sm_scale), _p(q),
                                _p(k), _p(v), _p(parent), _p(depth), _p(prefix_len),
                                _p(n_nodes), _p(out))
    return out


def kv_commit(k_all, v_all, prefix_len, accepted_nodes, n_accepted):
    """c2 (L635-644).  k_all/v_all [L][B][Hkv][Smax][D] uint16, modified in place, as is
    prefix_len (int32 [B])."""
    assert k_all.dtype == np.uint16 and k_all.flags.c_contiguous and v_all.flags.c_contiguous
    L, B, Hkv, Smax, D = k_all.shape
    accepted_nodes = _c(accepted_nodes, np.int32)
    n_accepted = _c(n_accepted, np.int32)
    assert prefix_len.dtype == np.int32 and prefix_len.flags.c_contiguous
    lib().oracle_kv_commit(L, B, Hkv, Smax, D, B * Hkv * Smax * D, accepted_nodes.shape[1],
                           _p(k_all), _p(v_all), _p(prefix_len), _p(accepted_nodes),
                           _p(n_accepted))


def verify_greedy(logits, tree_tokens, parent, n_nodes, *, depth=None, prefix_len=None,
                  smax=1 << 30, max_depth=255, path_len=None):
    """c3 (Alg. 2).  Returns (accepted_nodes, accepted_tokens, n_accepted)."""
    logits = _c(logits, np.float32)
    B, Nmax, V = logits.shape
    path_len = path_len or (max_depth + 1 if max_depth < 255 else Nmax + 1)
    an = np.empty((B, path_len), np.int32)
    at = np.empty((B, path_len), np.int32)
    na = np.empty((B,), np.int32)
    lib().oracle_verify_greedy(B, Nmax, V, smax, max_depth, path_len, _p(logits),
                               _p(_c(tree_tokens, np.int32)), _p(_c(parent, np.int32)),
                               _p(None if depth is None else _c(depth, np.int32)),
                               _p(None if prefix_len is None else _c(prefix_len, np.int32)),
                               _p(_c(n_nodes, np.int32)), _p(an), _p(at), _p(na))
    return an, at, na


class VerifyResult(tuple):
    """(accepted_nodes, accepted_tokens, n_accepted, margin) plus ``.decisions``: per request the
    list of decision records (node u, child s or -1 for a race, value, relative margin) in the
    order the sampler took them (c4's decision log)."""
    decisions: list


def _decision_log(B, stride):
    return (stride, np.full((B, stride), -1, np.int32), np.full((B, stride), -1, np.int32),
            np.full((B, stride), -1, np.int32), np.full((B, stride), np.inf), np.zeros((B,), np.int32))


def _result(an, at, na, mg, log):
    _, dn, dc, dv, dm, nd = log
    r = VerifyResult((an, at, na, mg))
    r.decisions = [[(int(dn[b, k]), int(dc[b, k]), int(dv[b, k]), float(dm[b, k])) for k in range(nd[b])]
                   for b in range(len(nd))]
    return r


def verify_mss(logits, tree_tokens, parent, n_nodes, draft_probs, *, temperature=1.0, seed=0,
               offset=0, request_ids=None, depth=None, prefix_len=None, smax=1 << 30,
               max_depth=255, path_len=None):
    """c4 (Alg. 2).  Returns (accepted_nodes, accepted_tokens, n_accepted, margin) with the
    per-decision log in ``.decisions`` (VerifyResult)."""
    logits = _c(logits, np.float32)
    draft_probs = _c(draft_probs, np.float32)
    B, Nmax, V = logits.shape
    assert draft_probs.shape == logits.shape
    path_len = path_len or (max_depth + 1 if max_depth < 255 else Nmax + 1)
    an = np.empty((B, path_len), np.int32)
    at = np.empty((B, path_len), np.int32)
    na = np.empty((B,), np.int32)
    mg = np.empty((B,), np.float64)
    rids = None if request_ids is None else _c(request_ids, np.int32)
    log = _decision_log(B, Nmax + 1)
    lib().oracle_verify_mss(B, Nmax, V, smax, max_depth, path_len, _p(logits),
                            _p(_c(tree_tokens, np.int32)), _p(_c(parent, np.int32)),
                            _p(None if depth is None else _c(depth, np.int32)),
                            _p(None if prefix_len is None else _c(prefix_len, np.int32)),
                            _p(_c(n_nodes, np.int32)), _p(draft_probs), float(temperature),
                            int(seed) & (2**64 - 1), int(offset) & (2**64 - 1), _p(rids),
                            _p(an), _p(at), _p(na), _p(mg), log[0], *[_p(a) for a in log[1:]])
    return _result(an, at, na, mg, log)


def verify_ns(logits, tree_tokens, parent, n_nodes, *, temperature=1.0, seed=0, offset=0, request_ids=None,
              depth=None, prefix_len=None, smax=1 << 30, max_depth=255, path_len=None):
    """NEXT-3 naive sampling (L747-753, the baseline of Theorem 4.3): x ~ p at each node by the
    exponential race (c4's counters at round 0); follow the child with token x, else stop.
    Returns (accepted_nodes, accepted_tokens, n_accepted, margin)."""
    logits = _c(logits, np.float32)
    B, Nmax, V = logits.shape
    path_len = path_len or (max_depth + 1 if max_depth < 255 else Nmax + 1)
    an = np.empty((B, path_len), np.int32)
    at = np.empty((B, path_len), np.int32)
    na = np.empty((B,), np.int32)
    mg = np.empty((B,), np.float64)
    rids = None if request_ids is None else _c(request_ids, np.int32)
    log = _decision_log(B, Nmax + 1)
    lib().oracle_verify_ns(B, Nmax, V, smax, max_depth, path_len, _p(logits), _p(_c(tree_tokens, np.int32)),
                           _p(_c(parent, np.int32)), _p(None if depth is None else _c(depth, np.int32)),
                           _p(None if prefix_len is None else _c(prefix_len, np.int32)),
                           _p(_c(n_nodes, np.int32)), float(temperature), int(seed) & (2**64 - 1),
                           int(offset) & (2**64 - 1), _p(rids), _p(an), _p(at), _p(na), _p(mg),
                           log[0], *[_p(a) for a in log[1:]])
    return _result(an, at, na, mg, log)


def philox4x32_10(ctr, key) -> np.ndarray:
    c = _c(ctr, np.uint32)
    k = _c(key, np.uint32)
    o = np.empty(4, np.uint32)
    lib().oracle_philox4x32_10(_p(c), _p(k), _p(o))
    return o


def leaf_paths(parent, n_nodes):
    """NEXT-1 (sequence-based decoding, §4.2, Fig. 4 left L682): the token
    tree decomposed into its root-to-leaf token sequences.  For each request: the leaves (nodes
    without children) in node-index order, each with the node ids of its path root .. leaf.
    Plain Python, literally the definition (a leaf is a node no other node names as parent;
    its sequence is the chain of parents up to the root).  Returns a list (per request) of lists
    of paths; an invalid tree (parent[0] != -1 or parent[i] not in [0, i)) gives None."""
    parent = np.asarray(parent)
    out = []
    for b in range(parent.shape[0]):
        n = int(n_nodes[b])
        par = [int(x) for x in parent[b, :n]]
        if n < 1 or par[0] != -1 or any(not (0 <= par[i] < i) for i in range(1, n)):
            out.append(None)
            continue
        has_child = set(par[1:])
        paths = []
        for leaf in range(n):
            if leaf in has_child:
                continue
            path = [leaf]
            while par[path[-1]] != -1:
                path.append(par[path[-1]])
            paths.append(path[::-1])
        out.append(paths)
    return out


# --------------------------------------------------------------------------------------------
# NEXT-2: token-tree construction (§3), plain Python by definition
# --------------------------------------------------------------------------------------------

def expansion_tree_bfs(expansion):
    """The static expansion <k1..km> (L476-483) built literally step by step: step i gives every
    node of the current frontier k_i children.  Returns (parent, depth) in BFS (creation) order."""
    parent, depth = [-1], [0]
    frontier = [0]
    for i, k in enumerate(expansion):
        nxt = []
        for u in frontier:
            for _ in range(k):
                parent.append(u)
                depth.append(i + 1)
                nxt.append(len(parent) - 1)
        frontier = nxt
    return parent, depth


def dfs_linearize(parent, tokens=None):
    """Depth-first linearisation (Fig. 2 "Linearization", L314): preorder, children in their order
    of creation.  Returns (new_parent, new_tokens, order) with order[new_id] = old_id."""
    n = len(parent)
    kids = [[] for _ in range(n)]
    for c in range(1, n):
        kids[parent[c]].append(c)
    order = []

    def visit(u):
        order.append(u)
        for c in kids[u]:
            visit(c)

    visit(0)
    new_id = {old: new for new, old in enumerate(order)}
    new_parent = [-1 if parent[o] < 0 else new_id[parent[o]] for o in order]
    new_tokens = None if tokens is None else [tokens[o] for o in order]
    return new_parent, new_tokens, order


def expand_topk(ssm_logits_row, k):
    """The k tokens of an SSM distribution expanded at a node (L455-468: its top-k), by a full
    sort: descending logit, lowest token id first among equals (reading R7)."""
    row = np.asarray(ssm_logits_row, np.float64)
    order = sorted(range(len(row)), key=lambda x: (-row[x], x))
    return order[:k]


def ssm_distribution(ssm_logits_row, temperature=1.0):
    """The SSM distribution a node's children are drawn from (L455-468; reading R12: the draft row
    of child c is the q that drew t_c), softmax(logits / T) in fp64, written out."""
    x = np.asarray(ssm_logits_row, np.float64) / float(temperature)
    e = np.exp(x - x.max())
    return e / e.sum()


def tree_merge(trees):
    """Token tree merge (Def. 3.2) by its definition: the set of sequences S_u of every
    input node (Def. 3.1: S_u = S_{p_u} + t_u) becomes one trie whose nodes are those sequences;
    children ordered by first appearance (inputs in order, nodes in index order); DFS preorder.
    `trees` = list of (parent, tokens).  Returns (parent, tokens, depth, node_maps) or None when
    the roots differ (all input roots are the same last verified token, reading R6)."""
    seqs = []          # distinct sequences in first-appearance order
    index = {}
    maps = []
    for par, tok in trees:
        S = []
        m = []
        for i in range(len(par)):
            s = (tuple(S[par[i]]) if par[i] >= 0 else ()) + (int(tok[i]),)
            S.append(list(s))
            if s not in index:
                index[s] = len(seqs)
                seqs.append(s)
            m.append(index[s])
        maps.append(m)
    if len({s[0] for s in seqs}) > 1:
        return None
    parent = [-1 if len(s) == 1 else index[s[:-1]] for s in seqs]
    tokens = [s[-1] for s in seqs]
    new_parent, new_tokens, order = dfs_linearize(parent, tokens)
    new_id = {old: new for new, old in enumerate(order)}
    depth = [len(seqs[o]) - 1 for o in order]
    return new_parent, new_tokens, depth, [[new_id[x] for x in m] for m in maps]


# --------------------------------------------------------------------------------------------
# NEXT-4: rotary position encoding of the tree at position P_b + depth[i] (SURVEY A4 / DESIGN R29)
# --------------------------------------------------------------------------------------------

def rope_inv_freq(head_dim=128, base=10000.0):
    """Rotary frequencies theta_i = base^(-2i/D), i < D/2, rounded to fp32 (the contract the CUDA
    path follows: fp32 table, fp32 angle pos * theta_i)."""
    i = np.arange(head_dim // 2, dtype=np.float64)
    return np.power(np.float64(base), -2.0 * i / head_dim).astype(np.float32)


def rope_rotate(x, pos, base=10000.0):
    """x [..., D] rotated at integer positions pos [...] (broadcast over the last axis), in fp64.
    Rotate-half pairing (dims i and i + D/2), as LLaMA: the angle a_i = fp32(pos) * theta_i is
    formed in fp32 (the contract), then x'_i = x_i cos a_i - x_{i+D/2} sin a_i and
    x'_{i+D/2} = x_{i+D/2} cos a_i + x_i sin a_i in fp64."""
    x = np.asarray(x, np.float64)
    D = x.shape[-1]
    th = rope_inv_freq(D, base)
    ang = (np.asarray(pos).astype(np.float32)[..., None] * th).astype(np.float64)  # fp32 product
    c, s = np.cos(ang), np.sin(ang)
    lo, hi = x[..., :D // 2], x[..., D // 2:]
    return np.concatenate([lo * c - hi * s, hi * c + lo * s], axis=-1)


def tree_rope(q, k_cache, prefix_len, depth, n_nodes, base=10000.0):
    """Reading A4: node i of request b sits at position P_b + depth[i] of its sequence S_u
    (Def. 4.1 L594-598 places u at index depth(u) after the committed prefix).  Rotates the tree
    queries q [B][Nmax][Hq][D] (rows i < n_b) and the tree keys k_cache [B][Hkv][Smax][D]
    (slots P_b + i, i < n_b) at that position; everything else is returned unchanged.
    Returns fp64 (q_rot, k_rot)."""
    q = np.array(q, np.float64)
    k = np.array(k_cache, np.float64)
    for b in range(q.shape[0]):
        P, n = int(prefix_len[b]), int(n_nodes[b])
        for i in range(n):
            pos = P + int(depth[b][i])
            q[b, i] = rope_rotate(q[b, i], np.full(q.shape[2], pos), base)
            k[b, :, P + i] = rope_rotate(k[b, :, P + i], np.full(k.shape[1], pos), base)
    return q, k
