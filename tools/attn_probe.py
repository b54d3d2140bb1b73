"""Tree-attention probe: per-launch time for a config and (optionally) the per-tile pipeline trace
of CTAs 0-7 (clock64 timestamps recorded by the kernel when a trace buffer is set).

    python tools/attn_probe.py [--config C2] [--layers 4] [--trace]
"""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import numpy as np
import torch

import paper_conf_asplos_miaoozcwzwzyssc24_b200 as spi
import workloads as W


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="C2")
    ap.add_argument("--layers", type=int, default=4)
    ap.add_argument("--batch", type=int, default=None)
    ap.add_argument("--prefix", type=int, default=None)
    ap.add_argument("--iters", type=int, default=20)
    ap.add_argument("--trace", action="store_true")
    ap.add_argument("--raw", action="store_true", help="with --trace: print the raw per-tile events")
    ap.add_argument("--expansion", default=None, help="override the tree: comma list <k1,..,km>")
    ap.add_argument("--lib", default=None, help="load this libspecinfer build instead (A/B experiments)")
    ap.add_argument("--flags", type=int, default=0, help="debug flags: 1 skip TMA, 2 skip MMA (timing only)")
    ap.add_argument("--early", action="store_true", help="SPECINFER_ATTN_EARLY_PREFIX on every launch but the "
                                                         "graph's first (as bench.py runs the layers)")
    a = ap.parse_args()
    if a.lib:
        spi.load_library(a.lib)
    elif a.trace or a.flags:
        from paper_conf_asplos_miaoozcwzwzyssc24_b200 import build_lib
        spi.load_library(build_lib.build(debug_hooks=True))  # hooks exist only in the development build
    cfg = W.CONFIGS[a.config]
    dev = torch.device("cuda:0")
    B = a.batch or cfg.batch
    P = a.prefix or cfg.prefix
    p, d = cfg.tree if not a.expansion else W.expansion_tree([int(x) for x in a.expansion.split(",")])
    tb = W.make_tree_batch([(p, d)] * B, [P] * B, device=dev, max_depth=max(cfg.max_depth, int(d.max())))
    smax = P + tb.max_nodes
    ai = W.make_attention_inputs(tb, a.layers, cfg.num_q_heads, cfg.num_kv_heads, smax, seed=1, device=dev)
    shape = spi.make_shape(B, tb.max_nodes, cfg.num_q_heads, cfg.num_kv_heads, smax, max_depth=cfg.max_depth)
    st = spi.TreeState.create(shape, tb.parent, tb.depth, tb.prefix_len, tb.n_nodes)
    st.prepare()
    out = torch.empty_like(ai.q)
    if a.flags:
        os.environ["SPECINFER_DEBUG_FLAGS"] = str(a.flags)
        spi.specinfer_debug_set_trace(None)
    for l in range(a.layers):
        st.attention(ai.q[l], ai.k_cache[l], ai.v_cache[l], out[l])
    torch.cuda.synchronize()
    # the launches are captured in a CUDA graph (as bench.py runs them): host call overhead excluded
    s = torch.cuda.Stream()
    s.wait_stream(torch.cuda.current_stream())
    g = torch.cuda.CUDAGraph()
    with torch.cuda.stream(s):
        with torch.cuda.graph(g, stream=s):
            for i in range(a.iters):
                l = i % a.layers
                st.attention(ai.q[l], ai.k_cache[l], ai.v_cache[l], out[l], prefetch=a.early and i > 0)
    torch.cuda.synchronize()
    g.replay()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    g.replay()
    e1.record()
    torch.cuda.synchronize()
    us = e0.elapsed_time(e1) * 1e3 / a.iters
    n = tb.n_nodes.cpu().numpy().astype(np.int64)
    pl = tb.prefix_len.cpu().numpy().astype(np.int64)
    byts = int(((pl + n) * cfg.num_kv_heads * 512).sum() + (n * cfg.num_q_heads * 512).sum())
    res = {"flags": a.flags, "config": a.config, "B": B, "P": P, "us_per_launch": round(us, 2), "GBps": round(byts / us / 1e3, 1)}
    print(json.dumps(res), flush=True)
    if a.trace:
        tr = torch.zeros(8 * 64 * 16 + 8 * 1024, dtype=torch.int64, device=dev)
        spi.specinfer_debug_set_trace(tr)
        st.attention(ai.q[0], ai.k_cache[0], ai.v_cache[0], out[0])
        torch.cuda.synchronize()
        spi.specinfer_debug_set_trace(None)
        allt = tr.cpu().numpy().astype(np.int64)
        t = allt[:8 * 64 * 16].reshape(8, 64, 16)
        kt = allt[8 * 64 * 16:].reshape(-1, 8)
        kt = kt[kt[:, 0] > 0]
        t0 = kt[:, 0].min() if len(kt) else 0
        if len(kt): print(f"kernel-level (us from first CTA entry) over {len(kt)} CTAs: entry max {(kt[:,0].max()-t0)/1e3:.2f}; "
              f"first K issue median {np.median(kt[:,2]-t0)/1e3:.2f} max {(kt[:,2].max()-t0)/1e3:.2f}; "
              f"exit min {(kt[:,1].min()-t0)/1e3:.2f} median {np.median(kt[:,1]-t0)/1e3:.2f} max {(kt[:,1].max()-t0)/1e3:.2f}")
        names = ["K-iss", "V-iss", "S-mma", "PV-mma", "sm-beg", "P-rdy", "epi-PV", "epi-end", "epi-st", "epi-ld", "seg-beg"]
        if a.raw:
            for c in range(2):
                x = t[c]
                base = x[0, 0]
                print(f"CTA {c} raw events (cycles rel. to first K issue): 0 K-iss 1 V-iss 2 S-mma 3 PV-mma 4/5 sm-beg g0/g1 6/7 P-rdy g0/g1 8 epi 9 epi-end")
                for i in range(40):
                    print(f"{i:3d} " + " ".join(f"{(v - base) if v else -1:8d}" for v in x[i, :12]))
            return
        for c in range(2):
            x = t[c]
            nv = int((x[:, 4] > 0).sum())
            base = x[0, 0]
            print(f"CTA {c}: {nv} tiles; cycles rel. to first K issue: " + " ".join(f"{n:>8s}" for n in names))
            for i in range(min(nv, 40)):
                print(f"{i:3d} " + " ".join(f"{(v - base) if v else -1:8d}" for v in x[i, :11]))
            busy = x[:nv, 5] - x[:nv, 4]
            per = np.diff(x[:nv, 5])
            lat = x[:nv, 2] - x[:nv, 0]
            epi = [(x[i + 1, 4] - x[i, 5]) for i in range(nv - 1) if x[i, 7] > 0]
            print(f"  softmax busy/tile median {np.median(busy):.0f}; P-ready period median {np.median(per):.0f} "
                  f"mean {np.mean(per):.0f}; K issue->S mma median {np.median(lat):.0f}; "
                  f"segment switch (P-ready -> next sm-begin) {epi}")
        np.save("gpurun_out/attn_trace.npy", t)


if __name__ == "__main__":
    main()
