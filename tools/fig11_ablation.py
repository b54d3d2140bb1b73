"""Synthetic Fig. 11 ablation (§6.5, Fig. 11): tree-based vs
sequence-based parallel decoding of the same token trees on B200, attention only.

For LLaMA-7B attention shapes (32 heads x 128, prefix P) and batch sizes 1..16 (Fig. 11), per
token tree (the paper's <1,1,k,1,1,1,1,1> of width k, L1078-1079):
  tree        one specinfer_tree_attention launch per layer (topology-aware mask, shared cache)
  seq-batch   one launch per layer over all root-to-leaf sequences, each with its own cache
              (specinfer_sequence_pack; the committed prefix is read once per leaf)
  seq-launch  one launch per sequence per layer (Fig. 4's Kernel 1/2/3)
Times are device times per layer from CUDA-graph replays of consecutive launches rotating over enough
layers' caches that every arm streams > 1 GB per replay (tools/graph_timing.py; host launch overhead
excluded, as in bench.py), x 32 layers.

    python tools/fig11_ablation.py [--prefix 2048] [--batches 1,2,4,8,16] [--widths 1,2,3,4,5]
Writes one JSON line per point to stdout (and to --out).
"""
import argparse
import json
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch

import paper_conf_asplos_miaoozcwzwzyssc24_b200 as spi
import workloads as W
from tools.graph_timing import graph_us_per_launch, layers_for


def timed(fn, iters, warm=3):
    for _ in range(warm):
        fn(0)
    torch.cuda.synchronize()
    ts = []
    for i in range(iters):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        fn(i)
        e1.record()
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1) * 1e3)
    return statistics.median(ts)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--prefix", type=int, default=2048)
    ap.add_argument("--batches", default="1,2,4,8,16")
    ap.add_argument("--widths", default="1,2,3,4,5")
    ap.add_argument("--layers", type=int, default=32)
    ap.add_argument("--iters", type=int, default=10)
    ap.add_argument("--out", default=None)
    a = ap.parse_args()
    dev = torch.device("cuda:0")
    H = 32
    rows = []
    for width in [int(x) for x in a.widths.split(",")]:
        expansion = (1, 1, width, 1, 1, 1, 1, 1)
        par, dep = W.expansion_tree(expansion)
        for B in [int(x) for x in a.batches.split(",")]:
            tb = W.make_tree_batch([(par, dep)] * B, [a.prefix] * B, device=dev, max_depth=len(expansion))
            smax = a.prefix + tb.max_nodes
            nl = layers_for(B * H * smax * 512, target=1 << 30, cap=8)
            ai = W.make_attention_inputs(tb, nl, H, H, smax, seed=11, device=dev)
            shape = spi.make_shape(B, tb.max_nodes, H, H, smax, max_depth=len(expansion))
            st = spi.TreeState.create(shape, tb.parent, tb.depth, tb.prefix_len, tb.n_nodes)
            st.prepare()
            out = torch.empty_like(ai.q[0])
            t_tree = graph_us_per_launch(lambda i, first: st.attention(ai.q[i % nl], ai.k_cache[i % nl],
                                                                       ai.v_cache[i % nl], out, prefetch=not first), nl)
            sbs = []
            for l in range(nl):
                sb = spi.SequenceBaseline(shape, tb.parent, tb.depth, tb.prefix_len, tb.n_nodes)
                sb.build(ai.q[l], ai.k_cache[l], ai.v_cache[l])
                sbs.append(sb)
            t_seq = graph_us_per_launch(lambda i, first: sbs[i % nl].attention(), nl)
            t_seql = graph_us_per_launch(lambda i, first: sbs[i % nl].attention(per_sequence=True), nl,
                                         reps=max(nl, 4))
            n = int(tb.n_nodes.sum())
            nseq = sbs[0].num_seqs
            kv_tree = B * H * (a.prefix + tb.max_nodes) * 512
            kv_seq = int((H * (a.prefix + sbs[0].seq_n.cpu().long()) * 512).sum())
            row = {"width": width, "expansion": list(expansion), "batch": B, "prefix": a.prefix, "tree_nodes": n // B,
                   "sequences": nseq, "sequence_query_rows": int(sbs[0].seq_n.sum()),
                   "us_per_layer": {"tree": round(t_tree, 2), "seq_batched": round(t_seq, 2),
                                    "seq_per_launch": round(t_seql, 2)},
                   "ms_per_iteration_32_layers": {"tree": round(t_tree * a.layers / 1e3, 3),
                                                  "seq_batched": round(t_seq * a.layers / 1e3, 3),
                                                  "seq_per_launch": round(t_seql * a.layers / 1e3, 3)},
                   "speedup_tree_vs_seq_batched": round(t_seq / t_tree, 3),
                   "speedup_tree_vs_seq_per_launch": round(t_seql / t_tree, 3),
                   "kv_bytes_per_layer": {"tree": kv_tree, "seq": kv_seq}}
            print(json.dumps(row), flush=True)
            rows.append(row)
            del sbs, ai
            torch.cuda.empty_cache()
    if a.out:
        with open(a.out, "w") as f:
            for r in rows:
                f.write(json.dumps(r) + "\n")


if __name__ == "__main__":
    main()
