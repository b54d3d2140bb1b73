"""Thin Python binding of libspecinfer.so (include/specinfer.h) — argument marshalling only.

SpecInfer's token-tree verification hot path on B200 (sm_100a): tree attention with the
topology-aware causal mask, greedy and multi-step-speculative-sampling verification, and the
depth-first KV-cache commit.  Every step runs in the hand-written CUDA kernels of the library;
PyTorch only provides device memory and streams.  There is no CPU fallback: if the library is
missing or the device is not sm_100, calls raise.

Function names are the C ABI names.  Tensors must be CUDA, contiguous, of the documented dtype
and shape; violations raise ValueError before anything is launched.
"""
from __future__ import annotations

import ctypes
import dataclasses
import os
from typing import Optional

import torch

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libspecinfer.so")
# development build with pipeline timestamps / experiment switches (build_lib.py --debug-hooks);
# tools load it explicitly with load_library(DEBUG_LIB_PATH); tests and the bench never do
DEBUG_LIB_PATH = os.path.join(_HERE, "libspecinfer_debug.so")

SPECINFER_OK = 0
STATUS_NAMES = {0: "OK", 1: "ERR_INVALID_ARG", 2: "ERR_UNSUPPORTED", 3: "ERR_CUDA", 4: "ERR_BAD_TREE",
                5: "ERR_WORKSPACE"}

EXPORTED_SYMBOLS = (
    "specinfer_workspace_size", "specinfer_tree_prepare", "specinfer_tree_attention",
    "specinfer_verify_greedy", "specinfer_verify_mss", "specinfer_kv_commit",
    "specinfer_read_device_status", "specinfer_philox_debug", "specinfer_debug_set_trace",
    "specinfer_launches_per_call",
    "specinfer_status_string", "specinfer_leaf_paths", "specinfer_sequence_pack",
    "specinfer_verify_ns", "specinfer_expansion_topology", "specinfer_expand_step", "specinfer_tree_merge",
    "specinfer_tree_attention_paged", "specinfer_kv_commit_paged", "specinfer_tree_rope",
    "specinfer_debug_hooks_enabled", "specinfer_tree_attention_ex", "specinfer_hbm_read_probe",
    "specinfer_verify_greedy_ex", "specinfer_verify_mss_ex", "specinfer_gather_wait",
)
MAX_PEERS = 8
SPECINFER_ATTN_EARLY_PREFIX = 1


class SpecInferError(RuntimeError):
    def __init__(self, call: str, status: int, msg: str):
        super().__init__(f"{call} failed: {STATUS_NAMES.get(status, status)} ({msg})")
        self.status = status


class Shape(ctypes.Structure):
    _fields_ = [("batch", ctypes.c_int32), ("max_nodes", ctypes.c_int32), ("num_q_heads", ctypes.c_int32),
                ("num_kv_heads", ctypes.c_int32), ("head_dim", ctypes.c_int32), ("max_seq", ctypes.c_int32),
                ("num_layers", ctypes.c_int32), ("vocab", ctypes.c_int32), ("max_depth", ctypes.c_int32),
                ("sm_scale", ctypes.c_float), ("layer_stride", ctypes.c_int64)]

    def __repr__(self):
        return "Shape(" + ", ".join(f"{n}={getattr(self, n)}" for n, _ in self._fields_) + ")"


class GatherDesc(ctypes.Structure):
    """specinfer_gather_t (NEXT-4a fused verify -> gather; include/specinfer.h)."""
    _fields_ = [("world", ctypes.c_int32), ("rank", ctypes.c_int32), ("rows_per_rank", ctypes.c_int32),
                ("row_len", ctypes.c_int32), ("recv", ctypes.c_void_p * MAX_PEERS),
                ("flags", ctypes.c_void_p * MAX_PEERS), ("state", ctypes.c_void_p)]


def make_shape(batch, max_nodes, num_q_heads, num_kv_heads, max_seq, *, num_layers=1, vocab=0,
               max_depth=None, sm_scale=0.0, layer_stride=0, head_dim=128) -> Shape:
    return Shape(batch, max_nodes, num_q_heads, num_kv_heads, head_dim, max_seq, num_layers, vocab,
                 max_nodes - 1 if max_depth is None else max_depth, float(sm_scale), layer_stride)


_lib = None


def load_library(path: str = LIB_PATH):
    """Loads libspecinfer.so (built by build_lib.py / __graft_entry__.build()).  Raises if absent."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(path):
        raise ImportError(f"{path} not found: build it with `python -m "
                          f"paper_conf_asplos_miaoozcwzwzyssc24_b200.build_lib` (no CPU fallback exists)")
    lib = ctypes.CDLL(path)
    vp, i32, u64, f32 = ctypes.c_void_p, ctypes.c_int32, ctypes.c_uint64, ctypes.c_float
    sp = ctypes.POINTER(Shape)
    lib.specinfer_workspace_size.argtypes = [sp]
    lib.specinfer_workspace_size.restype = ctypes.c_size_t
    lib.specinfer_tree_prepare.argtypes = [sp, vp, vp, vp, vp, vp, vp]
    lib.specinfer_tree_attention.argtypes = [sp, vp, vp, vp, vp, vp, vp, vp, vp, vp, vp]
    lib.specinfer_tree_attention_ex.argtypes = [sp, vp, vp, vp, vp, vp, vp, vp, vp, vp, ctypes.c_uint32, vp]
    lib.specinfer_verify_greedy.argtypes = [sp, vp, vp, vp, vp, vp, vp, vp, vp, vp]
    lib.specinfer_verify_mss.argtypes = [sp, vp, vp, vp, vp, vp, f32, u64, u64, vp, vp, vp, vp, vp, vp]
    lib.specinfer_kv_commit.argtypes = [sp, vp, vp, vp, vp, vp, vp]
    lib.specinfer_read_device_status.argtypes = [vp, vp, ctypes.POINTER(i32)]
    lib.specinfer_philox_debug.argtypes = [vp, vp, i32, vp]
    lib.specinfer_tree_attention_paged.argtypes = [sp, vp, vp, vp, i32, vp, vp, vp, vp, vp, vp, vp, vp]
    lib.specinfer_kv_commit_paged.argtypes = [sp, vp, vp, i32, vp, vp, vp, vp, vp]
    lib.specinfer_tree_rope.argtypes = [sp, vp, vp, vp, vp, vp, f32, vp]
    lib.specinfer_expansion_topology.argtypes = [sp, vp, i32, vp, vp, vp, vp]
    lib.specinfer_expand_step.argtypes = [sp, i32, i32, vp, f32, vp, vp, vp, vp, vp, vp, vp]
    lib.specinfer_tree_merge.argtypes = [sp, i32, i32, vp, vp, vp, vp, vp, vp, vp, vp, vp, vp]
    lib.specinfer_verify_ns.argtypes = [sp, vp, vp, vp, vp, f32, u64, u64, vp, vp, vp, vp, vp, vp]
    lib.specinfer_leaf_paths.argtypes = [sp, vp, vp, vp, vp, vp, vp, vp]
    lib.specinfer_sequence_pack.argtypes = [sp, i32, i32] + [vp] * 14 + [vp]
    lib.specinfer_debug_set_trace.argtypes = [vp]
    lib.specinfer_debug_set_trace.restype = None
    gp = ctypes.POINTER(GatherDesc)
    lib.specinfer_verify_greedy_ex.argtypes = [sp, vp, vp, vp, vp, vp, vp, vp, vp, gp, vp]
    lib.specinfer_verify_mss_ex.argtypes = [sp, vp, vp, vp, vp, vp, f32, u64, u64, vp, vp, vp, vp, vp, gp, vp]
    lib.specinfer_gather_wait.argtypes = [gp, vp, vp]
    for name in ("specinfer_verify_greedy_ex", "specinfer_verify_mss_ex", "specinfer_gather_wait"):
        getattr(lib, name).restype = i32
    lib.specinfer_hbm_read_probe.argtypes = [vp, ctypes.c_size_t, vp]
    lib.specinfer_hbm_read_probe.restype = i32
    lib.specinfer_debug_hooks_enabled.argtypes = []
    lib.specinfer_debug_hooks_enabled.restype = i32
    lib.specinfer_launches_per_call.argtypes = [ctypes.c_char_p]
    lib.specinfer_launches_per_call.restype = i32
    lib.specinfer_status_string.argtypes = [i32]
    lib.specinfer_status_string.restype = ctypes.c_char_p
    for name in ("specinfer_tree_prepare", "specinfer_tree_attention", "specinfer_tree_attention_ex",
                 "specinfer_verify_greedy",
                 "specinfer_verify_mss", "specinfer_kv_commit", "specinfer_read_device_status",
                 "specinfer_philox_debug", "specinfer_leaf_paths", "specinfer_sequence_pack", "specinfer_verify_ns",
                 "specinfer_expansion_topology", "specinfer_expand_step", "specinfer_tree_merge",
                 "specinfer_tree_attention_paged", "specinfer_kv_commit_paged", "specinfer_tree_rope"):
        getattr(lib, name).restype = i32
    _lib = lib
    return lib


def _check(call: str, status: int):
    if status != SPECINFER_OK:
        msg = load_library().specinfer_status_string(status).decode()
        raise SpecInferError(call, status, msg)


def _stream(t: torch.Tensor):
    return ctypes.c_void_p(torch.cuda.current_stream(t.device).cuda_stream)


def _req(name, t, dtype, shape=None, device=None):
    if not isinstance(t, torch.Tensor):
        raise ValueError(f"{name}: expected a torch.Tensor")
    if not t.is_cuda:
        raise ValueError(f"{name}: must be a CUDA tensor (no CPU path)")
    if t.dtype != dtype:
        raise ValueError(f"{name}: dtype {t.dtype}, expected {dtype}")
    if not t.is_contiguous():
        raise ValueError(f"{name}: must be contiguous")
    if shape is not None and tuple(t.shape) != tuple(shape):
        raise ValueError(f"{name}: shape {tuple(t.shape)}, expected {tuple(shape)}")
    if device is not None and t.device != device:
        raise ValueError(f"{name}: on {t.device}, expected {device}")
    return ctypes.c_void_p(t.data_ptr())


def _opt(name, t, dtype, shape, device):
    return None if t is None else _req(name, t, dtype, shape, device)


def specinfer_workspace_size(shape: Shape) -> int:
    return int(load_library().specinfer_workspace_size(ctypes.byref(shape)))


def alloc_workspace(shape: Shape, device) -> torch.Tensor:
    n = specinfer_workspace_size(shape)
    if n == 0:
        raise ValueError(f"unsupported shape {shape}")
    ws = torch.empty(n + 256, dtype=torch.uint8, device=device)
    off = (-ws.data_ptr()) % 256
    return ws[off:off + n]


def _tree_args(shape: Shape, parent, depth, prefix_len, n_nodes, dev):
    B, N = shape.batch, shape.max_nodes
    return (_req("parent", parent, torch.int32, (B, N), dev), _req("depth", depth, torch.int32, (B, N), dev),
            _req("prefix_len", prefix_len, torch.int32, (B,), dev), _req("n_nodes", n_nodes, torch.int32, (B,), dev))


def specinfer_tree_prepare(shape: Shape, parent, depth, prefix_len, n_nodes, workspace: torch.Tensor):
    dev = parent.device
    args = _tree_args(shape, parent, depth, prefix_len, n_nodes, dev)
    ws = _req("workspace", workspace, torch.uint8, None, dev)
    _check("specinfer_tree_prepare",
           load_library().specinfer_tree_prepare(ctypes.byref(shape), *args, ws, _stream(parent)))


def specinfer_tree_attention(shape: Shape, q, k_cache, v_cache, parent, depth, prefix_len, n_nodes,
                             out, workspace, flags: int = 0):
    """One layer of tree attention; flags != 0 calls specinfer_tree_attention_ex (include/specinfer.h:
    SPECINFER_ATTN_EARLY_PREFIX only when the previous kernel on the stream was not tree_prepare or
    kv_commit of this state)."""
    dev = q.device
    B, N, Hq, Hkv, S = shape.batch, shape.max_nodes, shape.num_q_heads, shape.num_kv_heads, shape.max_seq
    qp = _req("q", q, torch.bfloat16, (B, N, Hq, 128), dev)
    kp = _req("k_cache", k_cache, torch.bfloat16, (B, Hkv, S, 128), dev)
    vp = _req("v_cache", v_cache, torch.bfloat16, (B, Hkv, S, 128), dev)
    op = _req("out", out, torch.bfloat16, (B, N, Hq, 128), dev)
    args = _tree_args(shape, parent, depth, prefix_len, n_nodes, dev)
    ws = _req("workspace", workspace, torch.uint8, None, dev)
    lib = load_library()
    if flags:
        _check("specinfer_tree_attention_ex",
               lib.specinfer_tree_attention_ex(ctypes.byref(shape), qp, kp, vp, *args, op, ws, int(flags), _stream(q)))
    else:
        _check("specinfer_tree_attention",
               lib.specinfer_tree_attention(ctypes.byref(shape), qp, kp, vp, *args, op, ws, _stream(q)))


def specinfer_tree_attention_paged(shape: Shape, q, k_pages, v_pages, page_table, parent, depth, prefix_len, n_nodes,
                                   out, workspace):
    """NEXT-4: tree attention over a paged KV cache ([num_pages][Hkv][128][128] pages)."""
    dev = q.device
    B, N, Hq, Hkv = shape.batch, shape.max_nodes, shape.num_q_heads, shape.num_kv_heads
    npg = int(k_pages.shape[0])
    mp = (shape.max_seq + 127) // 128
    qp = _req("q", q, torch.bfloat16, (B, N, Hq, 128), dev)
    kp = _req("k_pages", k_pages, torch.bfloat16, (npg, Hkv, 128, 128), dev)
    vp_ = _req("v_pages", v_pages, torch.bfloat16, (npg, Hkv, 128, 128), dev)
    pt = _req("page_table", page_table, torch.int32, (B, mp), dev)
    op = _req("out", out, torch.bfloat16, (B, N, Hq, 128), dev)
    args = _tree_args(shape, parent, depth, prefix_len, n_nodes, dev)
    ws = _req("workspace", workspace, torch.uint8, None, dev)
    _check("specinfer_tree_attention_paged", load_library().specinfer_tree_attention_paged(
        ctypes.byref(shape), qp, kp, vp_, npg, pt, *args, op, ws, _stream(q)))


def specinfer_kv_commit_paged(shape: Shape, k_pages_all, v_pages_all, page_table, prefix_len, accepted_nodes,
                              n_accepted):
    """NEXT-4: KV commit on a paged cache ([L][num_pages][Hkv][128][128])."""
    dev = k_pages_all.device
    B, Lp = shape.batch, shape.max_depth + 1
    npg = int(k_pages_all.shape[-4])
    mp = (shape.max_seq + 127) // 128
    for nm, t in (("k_pages_all", k_pages_all), ("v_pages_all", v_pages_all)):
        _req(nm, t, torch.bfloat16, None, dev)
        stride = shape.layer_stride or npg * shape.num_kv_heads * 128 * 128
        if t.numel() < (shape.num_layers - 1) * stride + npg * shape.num_kv_heads * 128 * 128:
            raise ValueError(f"{nm}: too small for {shape.num_layers} layers")
    _check("specinfer_kv_commit_paged", load_library().specinfer_kv_commit_paged(
        ctypes.byref(shape), ctypes.c_void_p(k_pages_all.data_ptr()), ctypes.c_void_p(v_pages_all.data_ptr()), npg,
        _req("page_table", page_table, torch.int32, (B, mp), dev),
        _req("prefix_len", prefix_len, torch.int32, (B,), dev),
        _req("accepted_nodes", accepted_nodes, torch.int32, (B, Lp), dev),
        _req("n_accepted", n_accepted, torch.int32, (B,), dev), _stream(k_pages_all)))


def specinfer_tree_rope(shape: Shape, q, k_cache, prefix_len, depth, n_nodes, rope_base: float = 10000.0):
    """NEXT-4: rotary position encoding of the tree in place, node i at position P_b + depth[i]
    (reading A4).  q [B][Nmax][Hq][128] and/or k_cache [B][Hkv][Smax][128] (one layer; tree slots
    P_b + i), bf16; either may be None."""
    ref = q if q is not None else k_cache
    if ref is None:
        raise ValueError("specinfer_tree_rope: q and k_cache are both None")
    dev = ref.device
    B, N = shape.batch, shape.max_nodes
    _check("specinfer_tree_rope", load_library().specinfer_tree_rope(
        ctypes.byref(shape), _opt("q", q, torch.bfloat16, (B, N, shape.num_q_heads, 128), dev),
        _opt("k_cache", k_cache, torch.bfloat16, (B, shape.num_kv_heads, shape.max_seq, 128), dev),
        _req("prefix_len", prefix_len, torch.int32, (B,), dev), _req("depth", depth, torch.int32, (B, N), dev),
        _req("n_nodes", n_nodes, torch.int32, (B,), dev), float(rope_base), _stream(ref)))


def specinfer_verify_greedy(shape: Shape, logits, tree_tokens, parent, n_nodes, accepted_nodes,
                            accepted_tokens, n_accepted, workspace, gather: Optional[GatherDesc] = None):
    """VerifyGreedy; with `gather` (NEXT-4a) the accepted rows also go to every rank's receive table
    (specinfer_verify_greedy_ex)."""
    dev = logits.device
    B, N, V, Lp = shape.batch, shape.max_nodes, shape.vocab, shape.max_depth + 1
    args = (_req("logits", logits, torch.float32, (B, N, V), dev),
            _req("tree_tokens", tree_tokens, torch.int32, (B, N), dev),
            _req("parent", parent, torch.int32, (B, N), dev), _req("n_nodes", n_nodes, torch.int32, (B,), dev),
            _req("accepted_nodes", accepted_nodes, torch.int32, (B, Lp), dev),
            _req("accepted_tokens", accepted_tokens, torch.int32, (B, Lp), dev),
            _req("n_accepted", n_accepted, torch.int32, (B,), dev),
            _req("workspace", workspace, torch.uint8, None, dev))
    lib = load_library()
    if gather is not None:
        _check("specinfer_verify_greedy_ex",
               lib.specinfer_verify_greedy_ex(ctypes.byref(shape), *args, ctypes.byref(gather), _stream(logits)))
    else:
        _check("specinfer_verify_greedy", lib.specinfer_verify_greedy(ctypes.byref(shape), *args, _stream(logits)))


def specinfer_verify_mss(shape: Shape, logits, tree_tokens, parent, n_nodes, draft_probs, temperature,
                         seed, offset, request_ids, accepted_nodes, accepted_tokens, n_accepted, workspace,
                         gather: Optional[GatherDesc] = None):
    """VerifyStochastic (MSS); with `gather` the rows are also published (specinfer_verify_mss_ex)."""
    dev = logits.device
    B, N, V, Lp = shape.batch, shape.max_nodes, shape.vocab, shape.max_depth + 1
    if not (temperature > 0):
        raise ValueError("temperature must be > 0")
    a = (_req("logits", logits, torch.float32, (B, N, V), dev),
         _req("tree_tokens", tree_tokens, torch.int32, (B, N), dev),
         _req("parent", parent, torch.int32, (B, N), dev), _req("n_nodes", n_nodes, torch.int32, (B,), dev),
         _req("draft_probs", draft_probs, torch.float32, (B, N, V), dev))
    rid = _opt("request_ids", request_ids, torch.int32, (B,), dev)
    o = (_req("accepted_nodes", accepted_nodes, torch.int32, (B, Lp), dev),
         _req("accepted_tokens", accepted_tokens, torch.int32, (B, Lp), dev),
         _req("n_accepted", n_accepted, torch.int32, (B,), dev),
         _req("workspace", workspace, torch.uint8, None, dev))
    lib = load_library()
    sc = (ctypes.c_float(temperature), ctypes.c_uint64(int(seed) & (2**64 - 1)),
          ctypes.c_uint64(int(offset) & (2**64 - 1)), rid)
    if gather is not None:
        _check("specinfer_verify_mss_ex",
               lib.specinfer_verify_mss_ex(ctypes.byref(shape), *a, *sc, *o, ctypes.byref(gather), _stream(logits)))
    else:
        _check("specinfer_verify_mss", lib.specinfer_verify_mss(ctypes.byref(shape), *a, *sc, *o, _stream(logits)))


def specinfer_gather_wait(gather: GatherDesc, table_out: Optional[torch.Tensor] = None, stream_of=None):
    """NEXT-4a: wait for every rank's rows of this step, copy them to `table_out` (int32
    [world * rows_per_rank][row_len], CUDA), advance the epoch.  Stream: the current stream of
    `table_out`'s device (or of `stream_of`)."""
    ref = table_out if table_out is not None else stream_of
    if ref is None:
        raise ValueError("specinfer_gather_wait: pass table_out or stream_of (a CUDA tensor)")
    tp = None
    if table_out is not None:
        tp = _req("table_out", table_out, torch.int32, (gather.world * gather.rows_per_rank, gather.row_len),
                  table_out.device)
    _check("specinfer_gather_wait", load_library().specinfer_gather_wait(ctypes.byref(gather), tp, _stream(ref)))


def specinfer_verify_ns(shape: Shape, logits, tree_tokens, parent, n_nodes, temperature, seed, offset, request_ids,
                        accepted_nodes, accepted_tokens, n_accepted, workspace):
    """NEXT-3 naive sampling (L747-753), see include/specinfer.h."""
    dev = logits.device
    B, N, V, Lp = shape.batch, shape.max_nodes, shape.vocab, shape.max_depth + 1
    if not (temperature > 0):
        raise ValueError("temperature must be > 0")
    a = (_req("logits", logits, torch.float32, (B, N, V), dev),
         _req("tree_tokens", tree_tokens, torch.int32, (B, N), dev),
         _req("parent", parent, torch.int32, (B, N), dev), _req("n_nodes", n_nodes, torch.int32, (B,), dev))
    rid = _opt("request_ids", request_ids, torch.int32, (B,), dev)
    o = (_req("accepted_nodes", accepted_nodes, torch.int32, (B, Lp), dev),
         _req("accepted_tokens", accepted_tokens, torch.int32, (B, Lp), dev),
         _req("n_accepted", n_accepted, torch.int32, (B,), dev),
         _req("workspace", workspace, torch.uint8, None, dev))
    _check("specinfer_verify_ns",
           load_library().specinfer_verify_ns(ctypes.byref(shape), *a, ctypes.c_float(temperature),
                                              ctypes.c_uint64(int(seed) & (2**64 - 1)),
                                              ctypes.c_uint64(int(offset) & (2**64 - 1)), rid, *o, _stream(logits)))


def specinfer_kv_commit(shape: Shape, k_cache_all, v_cache_all, prefix_len, accepted_nodes, n_accepted):
    dev = k_cache_all.device
    B, Lp = shape.batch, shape.max_depth + 1
    for nm, t in (("k_cache_all", k_cache_all), ("v_cache_all", v_cache_all)):
        _req(nm, t, torch.bfloat16, None, dev)
        stride = shape.layer_stride or B * shape.num_kv_heads * shape.max_seq * 128
        if t.numel() < (shape.num_layers - 1) * stride + B * shape.num_kv_heads * shape.max_seq * 128:
            raise ValueError(f"{nm}: too small for {shape.num_layers} layers")
    _check("specinfer_kv_commit", load_library().specinfer_kv_commit(
        ctypes.byref(shape), ctypes.c_void_p(k_cache_all.data_ptr()), ctypes.c_void_p(v_cache_all.data_ptr()),
        _req("prefix_len", prefix_len, torch.int32, (B,), dev),
        _req("accepted_nodes", accepted_nodes, torch.int32, (B, Lp), dev),
        _req("n_accepted", n_accepted, torch.int32, (B,), dev), _stream(k_cache_all)))


def specinfer_read_device_status(workspace: torch.Tensor) -> int:
    """Synchronises the current stream; returns the status bits (bit 0 = some tree invalid)."""
    bits = ctypes.c_int32(0)
    st = load_library().specinfer_read_device_status(ctypes.c_void_p(workspace.data_ptr()), _stream(workspace),
                                                    ctypes.byref(bits))
    if st not in (0, 4):
        _check("specinfer_read_device_status", st)
    return int(bits.value)


def specinfer_philox_debug(ctr_key: torch.Tensor) -> torch.Tensor:
    """ctr_key int64/uint32-valued tensor [n][6] -> [n][4] uint32 words as int64 (device Philox)."""
    dev = ctr_key.device
    ck = ctr_key.to(torch.int64).bitwise_and(0xFFFFFFFF).to(torch.int32).contiguous()
    out = torch.empty((ck.shape[0], 4), dtype=torch.int32, device=dev)
    _check("specinfer_philox_debug", load_library().specinfer_philox_debug(
        ctypes.c_void_p(ck.data_ptr()), ctypes.c_void_p(out.data_ptr()), ck.shape[0], _stream(ck)))
    return out.to(torch.int64).bitwise_and(0xFFFFFFFF)


def specinfer_expansion_topology(shape: Shape, expansion, parent, depth, n_nodes):
    """NEXT-2: the static expansion tree <k1..km> for every request (DFS preorder)."""
    dev = parent.device
    B, N = shape.batch, shape.max_nodes
    ks = (ctypes.c_int32 * len(expansion))(*[int(k) for k in expansion])
    _check("specinfer_expansion_topology", load_library().specinfer_expansion_topology(
        ctypes.byref(shape), ks, len(expansion), _req("parent", parent, torch.int32, (B, N), dev),
        _req("depth", depth, torch.int32, (B, N), dev), _req("n_nodes", n_nodes, torch.int32, (B,), dev),
        _stream(parent)))


def specinfer_expand_step(shape: Shape, level: int, ssm_logits, temperature, parent, depth, n_nodes, tree_tokens,
                          draft_probs=None, workspace=None):
    """NEXT-2: one expansion step (top-k of each frontier node's SSM logits -> its children)."""
    dev = ssm_logits.device
    B, N, V = shape.batch, shape.max_nodes, shape.vocab
    F = int(ssm_logits.shape[1])
    if not (temperature > 0):
        raise ValueError("temperature must be > 0")
    args = (_req("ssm_logits", ssm_logits, torch.float32, (B, F, V), dev),)
    _check("specinfer_expand_step", load_library().specinfer_expand_step(
        ctypes.byref(shape), int(level), F, *args, ctypes.c_float(temperature),
        _req("parent", parent, torch.int32, (B, N), dev), _req("depth", depth, torch.int32, (B, N), dev),
        _req("n_nodes", n_nodes, torch.int32, (B,), dev), _req("tree_tokens", tree_tokens, torch.int32, (B, N), dev),
        _opt("draft_probs", draft_probs, torch.float32, (B, N, V), dev),
        _opt("workspace", workspace, torch.uint8, None, dev), _stream(ssm_logits)))


def specinfer_tree_merge(shape: Shape, in_parent, in_tokens, in_n, parent, depth, tree_tokens, n_nodes, node_map,
                         workspace=None):
    """NEXT-2: token tree merge (Def. 3.2) of [B][T][Nin] input trees into [B][Nmax] DFS trees."""
    dev = in_parent.device
    B, N = shape.batch, shape.max_nodes
    T, Nin = int(in_parent.shape[1]), int(in_parent.shape[2])
    _check("specinfer_tree_merge", load_library().specinfer_tree_merge(
        ctypes.byref(shape), T, Nin, _req("in_parent", in_parent, torch.int32, (B, T, Nin), dev),
        _req("in_tokens", in_tokens, torch.int32, (B, T, Nin), dev), _req("in_n", in_n, torch.int32, (B, T), dev),
        _req("parent", parent, torch.int32, (B, N), dev), _req("depth", depth, torch.int32, (B, N), dev),
        _req("tree_tokens", tree_tokens, torch.int32, (B, N), dev), _req("n_nodes", n_nodes, torch.int32, (B,), dev),
        _req("node_map", node_map, torch.int32, (B, T, Nin), dev),
        _opt("workspace", workspace, torch.uint8, None, dev), _stream(in_parent)))


def specinfer_leaf_paths(shape: Shape, parent, n_nodes, paths, path_len, n_leaves, workspace=None):
    """NEXT-1: leaves (node-index order) and their root paths, see include/specinfer.h."""
    dev = parent.device
    B, N, Lp = shape.batch, shape.max_nodes, shape.max_depth + 1
    args = (_req("parent", parent, torch.int32, (B, N), dev), _req("n_nodes", n_nodes, torch.int32, (B,), dev),
            _req("paths", paths, torch.int32, (B, N, Lp), dev), _req("path_len", path_len, torch.int32, (B, N), dev),
            _req("n_leaves", n_leaves, torch.int32, (B,), dev),
            _opt("workspace", workspace, torch.uint8, None, dev))
    _check("specinfer_leaf_paths", load_library().specinfer_leaf_paths(ctypes.byref(shape), *args, _stream(parent)))


def specinfer_sequence_pack(shape: Shape, seq_map, paths, path_len, prefix_len, q, k_cache, v_cache, q_seq, k_seq,
                            v_seq, seq_parent, seq_depth, seq_prefix_len, seq_n_nodes):
    """NEXT-1: the per-sequence caches / queries / chain trees of sequence-based decoding (one
    layer), see include/specinfer.h."""
    dev = q.device
    B, N, Hq, Hkv, S, Lp = (shape.batch, shape.max_nodes, shape.num_q_heads, shape.num_kv_heads, shape.max_seq,
                            shape.max_depth + 1)
    ns = int(seq_map.shape[0])
    sms = int(k_seq.shape[2])
    args = (_req("seq_map", seq_map, torch.int32, (ns, 2), dev), _req("paths", paths, torch.int32, (B, N, Lp), dev),
            _req("path_len", path_len, torch.int32, (B, N), dev),
            _req("prefix_len", prefix_len, torch.int32, (B,), dev),
            _req("q", q, torch.bfloat16, (B, N, Hq, 128), dev),
            _req("k_cache", k_cache, torch.bfloat16, (B, Hkv, S, 128), dev),
            _req("v_cache", v_cache, torch.bfloat16, (B, Hkv, S, 128), dev),
            _req("q_seq", q_seq, torch.bfloat16, (ns, Lp, Hq, 128), dev),
            _req("k_seq", k_seq, torch.bfloat16, (ns, Hkv, sms, 128), dev),
            _req("v_seq", v_seq, torch.bfloat16, (ns, Hkv, sms, 128), dev),
            _req("seq_parent", seq_parent, torch.int32, (ns, Lp), dev),
            _req("seq_depth", seq_depth, torch.int32, (ns, Lp), dev),
            _req("seq_prefix_len", seq_prefix_len, torch.int32, (ns,), dev),
            _req("seq_n_nodes", seq_n_nodes, torch.int32, (ns,), dev))
    _check("specinfer_sequence_pack", load_library().specinfer_sequence_pack(
        ctypes.byref(shape), ns, sms, *args, _stream(q)))


def specinfer_debug_set_trace(trace: Optional[torch.Tensor]):
    """Debug only: per-tile timestamps of tree_attention CTAs 0-7 into `trace` (int64 [8][64][8])."""
    load_library().specinfer_debug_set_trace(None if trace is None else ctypes.c_void_p(trace.data_ptr()))


def specinfer_hbm_read_probe(buf: torch.Tensor):
    """Streams every byte of the CUDA tensor `buf` through the library's TMA read probe (measurement)."""
    if not isinstance(buf, torch.Tensor) or not buf.is_cuda or not buf.is_contiguous():
        raise ValueError("specinfer_hbm_read_probe: needs a contiguous CUDA tensor")
    nbytes = buf.numel() * buf.element_size()
    _check("specinfer_hbm_read_probe", load_library().specinfer_hbm_read_probe(
        ctypes.c_void_p(buf.data_ptr()), ctypes.c_size_t(nbytes), _stream(buf)))


def specinfer_launches_per_call(name: str) -> int:
    return int(load_library().specinfer_launches_per_call(name.encode()))


# ------------------------------------------------------------------------------------------
# convenience: a prepared verification iteration (used by bench.py and the tests)
# ------------------------------------------------------------------------------------------

@dataclasses.dataclass
class TreeState:
    shape: Shape
    parent: torch.Tensor
    depth: torch.Tensor
    prefix_len: torch.Tensor
    n_nodes: torch.Tensor
    workspace: torch.Tensor

    @classmethod
    def create(cls, shape: Shape, parent, depth, prefix_len, n_nodes, workspace=None):
        ws = workspace if workspace is not None else alloc_workspace(shape, parent.device)
        return cls(shape, parent, depth, prefix_len, n_nodes, ws)

    def prepare(self):
        specinfer_tree_prepare(self.shape, self.parent, self.depth, self.prefix_len, self.n_nodes, self.workspace)

    def attention(self, q, k, v, out, prefetch: bool = False):
        """prefetch=True: SPECINFER_ATTN_EARLY_PREFIX (the previous kernel on the stream was another
        attention layer, not prepare / commit)."""
        specinfer_tree_attention(self.shape, q, k, v, self.parent, self.depth, self.prefix_len, self.n_nodes,
                                 out, self.workspace, flags=SPECINFER_ATTN_EARLY_PREFIX if prefetch else 0)


# ------------------------------------------------------------------------------------------
# NEXT-1: sequence-based parallel decoding (the baseline of PAPER.md §4.2 / Fig. 4 left)
# ------------------------------------------------------------------------------------------

class SequenceBaseline:
    """Sequence-based parallel decoding of a tree batch (Fig. 4 left, §6.5):
    every root-to-leaf sequence gets its own KV cache (committed prefix + its own tokens) and is
    decoded as a causal chain.  `build()` decomposes the trees and packs one layer's caches
    (specinfer_leaf_paths + specinfer_sequence_pack); `attention()` runs all sequences in one
    tree_attention launch over chain trees, or one launch per sequence (`per_sequence=True`,
    Fig. 4's Kernel 1/2/3).  Only the host reads n_leaves (once, to size the sequence batch)."""

    def __init__(self, shape: Shape, parent, depth, prefix_len, n_nodes):
        dev = parent.device
        B, N, Lp = shape.batch, shape.max_nodes, shape.max_depth + 1
        self.tree_shape = shape
        self.prefix_len = prefix_len
        self.paths = torch.empty((B, N, Lp), dtype=torch.int32, device=dev)
        self.path_len = torch.empty((B, N), dtype=torch.int32, device=dev)
        self.n_leaves = torch.empty((B,), dtype=torch.int32, device=dev)
        specinfer_leaf_paths(shape, parent, n_nodes, self.paths, self.path_len, self.n_leaves)
        nl = self.n_leaves.cpu().tolist()
        self.seq_map = torch.tensor([(b, r) for b in range(B) for r in range(nl[b])], dtype=torch.int32,
                                    device=dev).reshape(-1, 2)
        ns = int(self.seq_map.shape[0])
        self.num_seqs = ns
        pmax = int(prefix_len.max().item())
        self.seq_max_seq = pmax + Lp
        Hq, Hkv = shape.num_q_heads, shape.num_kv_heads
        self.shape = make_shape(ns, Lp, Hq, Hkv, self.seq_max_seq, max_depth=shape.max_depth,
                                sm_scale=shape.sm_scale)
        self.q = torch.empty((ns, Lp, Hq, 128), dtype=torch.bfloat16, device=dev)
        self.k = torch.empty((ns, Hkv, self.seq_max_seq, 128), dtype=torch.bfloat16, device=dev)
        self.v = torch.empty_like(self.k)
        self.out = torch.empty_like(self.q)
        self.parent = torch.empty((ns, Lp), dtype=torch.int32, device=dev)
        self.depth = torch.empty_like(self.parent)
        self.seq_prefix = torch.empty((ns,), dtype=torch.int32, device=dev)
        self.seq_n = torch.empty_like(self.seq_prefix)
        self.state = None
        self.singles = None  # per-sequence states (per_sequence=True), prepared once

    def build(self, q, k_cache, v_cache):
        specinfer_sequence_pack(self.tree_shape, self.seq_map, self.paths, self.path_len, self.prefix_len, q,
                                k_cache, v_cache, self.q, self.k, self.v, self.parent, self.depth, self.seq_prefix,
                                self.seq_n)
        if self.state is None:
            self.state = TreeState.create(self.shape, self.parent, self.depth, self.seq_prefix, self.seq_n)
        self.state.prepare()

    def attention(self, per_sequence: bool = False):
        if not per_sequence:
            self.state.attention(self.q, self.k, self.v, self.out)
            return self.out
        if self.singles is None:
            s1 = make_shape(1, self.shape.max_nodes, self.shape.num_q_heads, self.shape.num_kv_heads,
                            self.seq_max_seq, max_depth=self.shape.max_depth, sm_scale=self.shape.sm_scale)
            self.singles = []
            for s in range(self.num_seqs):
                st = TreeState.create(s1, self.parent[s:s + 1], self.depth[s:s + 1], self.seq_prefix[s:s + 1],
                                      self.seq_n[s:s + 1])
                st.prepare()
                self.singles.append(st)
        for s, st in enumerate(self.singles):
            st.attention(self.q[s:s + 1], self.k[s:s + 1], self.v[s:s + 1], self.out[s:s + 1])
        return self.out
