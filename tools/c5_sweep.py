"""Config C5 (BASELINE.json configs[4]): tree size x batch x prefix sweep of the tree-attention
kernel (one layer per point, LLaMA-7B heads 32 x 128 MHA) and of greedy verification (V = 32000),
each point reported against the HBM and the tensor roofline.

    python tools/c5_sweep.py [--out gpurun_out/c5_sweep.jsonl] [--iters 10] [--quick]

Per point: random trees of exactly n nodes (depth <= 8, fanout <= 8, DFS preorder, seeded), prefix P
for every request.  Attention timing: a CUDA graph of consecutive launches (as bench.py runs the layers:
SPECINFER_ATTN_EARLY_PREFIX after the first) rotating over enough layers' caches that the streamed bytes
exceed 512 MB (4x the L2), per-launch = graph time / launches (tools/graph_timing.py).  Verification:
CUDA events around each launch with a 256 MB L2 flush before it.  Roofline denominators: the driver's
MEASURED_PEAKS.json (hbm_gbs; bf16 sustained for tensor-bound points), else the guide's fallback.  Algorithmic bytes per (request, kv-head) = (P + n)*128*2*2
(K, V read once) + G*n*128*2*2 (q in, out); FLOPs per (request, q-head) = 4*128*(n*P + sum(depth+1)).
"""
import argparse
import json
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import numpy as np
import torch

import paper_conf_asplos_miaoozcwzwzyssc24_b200 as spi
import workloads as W
from tools.graph_timing import graph_us_per_launch, layers_for


def peaks():
    try:
        d = json.load(open(os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))),
                                        "MEASURED_PEAKS.json")))
        return float(d["hbm_gbs"]), float(d.get("bf16_tflops_sustained", d["bf16_tflops"])), "measured"
    except Exception:
        return 6650.0, 1590.0, "fallback"


def timed(fn, flush, iters):
    stream = torch.cuda.current_stream()
    ts = []
    for _ in range(iters):
        flush.zero_()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        fn()
        e1.record(stream)
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1) * 1e3)
    return statistics.median(ts)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--out", default="gpurun_out/c5_sweep.jsonl")
    ap.add_argument("--iters", type=int, default=10)
    ap.add_argument("--heads", type=int, default=32)
    ap.add_argument("--vocab", type=int, default=32000)
    ap.add_argument("--quick", action="store_true", help="a 6-point subset")
    a = ap.parse_args()
    dev = torch.device("cuda:0")
    torch.cuda.set_device(dev)
    hbm, tf, src = peaks()
    H = a.heads
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)
    pts = W.c5_points()
    if a.quick:
        pts = [(8, 1, 512), (21, 16, 2048), (64, 8, 2048), (128, 64, 2048), (256, 8, 8192), (256, 64, 8192)]
    os.makedirs(os.path.dirname(a.out) or ".", exist_ok=True)
    fo = open(a.out, "w")
    for (n, B, P) in pts:
        tb = W.random_tree_batch(B, n, P, seed=1000 + n, device=dev)
        smax = P + n
        nl = layers_for(B * H * smax * 512)
        ai = W.make_attention_inputs(tb, nl, H, H, smax, seed=5, device=dev)
        shape = spi.make_shape(B, tb.max_nodes, H, H, smax, vocab=a.vocab, max_depth=tb.max_depth)
        st = spi.TreeState.create(shape, tb.parent, tb.depth, tb.prefix_len, tb.n_nodes)
        st.prepare()
        out = torch.empty_like(ai.q[0])
        us = graph_us_per_launch(lambda i, first: st.attention(ai.q[i % nl], ai.k_cache[i % nl], ai.v_cache[i % nl],
                                                               out, prefetch=not first), nl)
        # greedy verification of the same trees (logits fp32 [B][n][V])
        vi = W.make_verify_inputs(tb, a.vocab, seed=5, mode="greedy", device=dev)
        an = torch.empty((B, tb.max_depth + 1), dtype=torch.int32, device=dev)
        at = torch.empty_like(an)
        na = torch.empty((B,), dtype=torch.int32, device=dev)
        run_v = lambda: spi.specinfer_verify_greedy(shape, vi.logits, vi.tree_tokens, tb.parent, tb.n_nodes,
                                                    an, at, na, st.workspace)
        for _ in range(3):
            run_v()
        us_v = timed(run_v, flush, a.iters)
        nn = tb.n_nodes.cpu().numpy().astype(np.int64)
        pl = tb.prefix_len.cpu().numpy().astype(np.int64)
        dep = tb.depth.cpu().numpy().astype(np.int64)
        anc_pairs = sum(int((dep[b, :nn[b]] + 1).sum()) for b in range(B))
        byts = int(((pl + nn) * H * 512).sum() + (nn * H * 512).sum())
        flops = 4 * 128 * H * (int((nn * pl).sum()) + anc_pairs)
        vbytes = int(nn.sum()) * a.vocab * 4
        gbs = byts / us / 1e3
        tfs = flops / us / 1e6
        ai_ = flops / byts
        bound = "tensor" if ai_ > tf * 1e3 / hbm else "hbm"
        rec = {"n": n, "batch": B, "prefix": P, "attn_us": round(us, 2), "attn_GBps": round(gbs, 1),
               "hbm_frac": round(gbs / hbm, 4), "attn_TFps": round(tfs, 1), "tensor_frac": round(tfs / tf, 4),
               "AI": round(ai_, 1), "bound": bound,
               "roofline_frac": round(gbs / hbm if bound == "hbm" else tfs / tf, 4),
               "verify_greedy_us": round(us_v, 2), "verify_GBps": round(vbytes / us_v / 1e3, 1),
               "tree_tok_per_s_per_layer": round(int(nn.sum()) / (us * 1e-6), 1), "graph_layers": nl,
               "peaks": {"hbm_gbs": hbm, "bf16_tflops": tf, "source": src}}
        print(json.dumps(rec), flush=True)
        fo.write(json.dumps(rec) + "\n")
        fo.flush()
        del ai, vi, st, out
        torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
