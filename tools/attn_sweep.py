"""Tree-attention rate vs tree size (development tool): one layer, LLaMA-7B heads (32 x 128, MHA),
random trees of exactly n nodes (depth <= 8), batch B, prefix P; CUDA-event time per launch and the
achieved algorithmic GB/s (K/V read once + q/out), two cache copies alternating.

    python tools/attn_sweep.py [--ns 8,16,21,27,32,33,48,64,65,96,128] [--batch 16] [--prefix 2048]
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


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--ns", default="8,16,21,27,32,33,48,64,65,96,128")
    ap.add_argument("--batch", type=int, default=16)
    ap.add_argument("--prefix", type=int, default=2048)
    ap.add_argument("--heads", type=int, default=32)
    ap.add_argument("--iters", type=int, default=20)
    ap.add_argument("--lib", default=None, help="load this libspecinfer build instead (A/B experiments)")
    a = ap.parse_args()
    if a.lib:
        spi.load_library(a.lib)
    dev = torch.device("cuda:0")
    H = a.heads
    for n in [int(x) for x in a.ns.split(",")]:
        tb = W.random_tree_batch(a.batch, n, a.prefix, seed=n, device=dev)
        smax = a.prefix + n
        ai = W.make_attention_inputs(tb, 2, H, H, smax, seed=3, device=dev)
        shape = spi.make_shape(a.batch, tb.max_nodes, H, H, smax, max_depth=tb.max_depth)
        st = spi.TreeState.create(shape, tb.parent, tb.depth, tb.prefix_len, tb.n_nodes)
        st.prepare()
        out = torch.empty_like(ai.q[0])
        for i in range(3):
            st.attention(ai.q[i & 1], ai.k_cache[i & 1], ai.v_cache[i & 1], out)
        torch.cuda.synchronize()
        ts = []
        for i in range(a.iters):
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            st.attention(ai.q[i & 1], ai.k_cache[i & 1], ai.v_cache[i & 1], out)
            e1.record()
            torch.cuda.synchronize()
            ts.append(e0.elapsed_time(e1) * 1e3)
        us = statistics.median(ts)
        nn = tb.n_nodes.cpu().numpy().astype(np.int64)
        pl = tb.prefix_len.cpu().numpy().astype(np.int64)
        byts = int(((pl + nn) * H * 512).sum() + (nn * H * 512).sum())
        print(json.dumps({"n": n, "batch": a.batch, "prefix": a.prefix, "us": round(us, 2),
                          "GBps": round(byts / us / 1e3, 1)}), flush=True)
        del ai
        torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
