"""Step-segment probe (development tool): device time per launch of the small kernels of a bench
step at a config / batch, each repeated inside one CUDA graph (tools/graph_timing.py), plus the
same chain with a torch copy in front (the bench's per-step prefix reset).

    python tools/step_probe.py --config C1 [--batch 2] [--lib path]
"""
import argparse
import dataclasses
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import paper_conf_asplos_miaoozcwzwzyssc24_b200 as spi
import workloads as W
from tools.graph_timing import graph_us_per_launch


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="C1")
    ap.add_argument("--batch", type=int, default=None)
    ap.add_argument("--lib", default=None)
    a = ap.parse_args()
    if a.lib:
        spi.load_library(a.lib)
    cfg = W.CONFIGS[a.config]
    if a.batch:
        cfg = dataclasses.replace(cfg, batch=a.batch)
    dev = torch.device("cuda:0")
    tb = W.config_tree_batch(cfg, device=dev)
    B, Lp = cfg.batch, cfg.max_depth + 1
    smax = cfg.prefix + tb.max_nodes
    shape = spi.make_shape(B, tb.max_nodes, cfg.num_q_heads, cfg.num_kv_heads, smax, vocab=cfg.vocab,
                           max_depth=cfg.max_depth, num_layers=1)
    st = spi.TreeState.create(shape, tb.parent, tb.depth, tb.prefix_len, tb.n_nodes)
    st.prepare()
    p0 = tb.prefix_len.clone()
    res = {"config": a.config, "batch": B}
    res["prepare_us"] = round(graph_us_per_launch(lambda i, f: st.prepare(), 1, reps=32), 2)
    res["copy+prepare_us"] = round(graph_us_per_launch(lambda i, f: (tb.prefix_len.copy_(p0), st.prepare()), 1,
                                                       reps=32), 2)
    print(json.dumps(res), flush=True)
    vi = W.make_verify_inputs(tb, cfg.vocab, seed=cfg.seed, mode="greedy", device=dev)
    an = torch.empty((B, Lp), dtype=torch.int32, device=dev)
    at, na = torch.empty_like(an), torch.empty((B,), dtype=torch.int32, device=dev)
    res["verify_greedy_us"] = round(graph_us_per_launch(
        lambda i, f: spi.specinfer_verify_greedy(shape, vi.logits, vi.tree_tokens, tb.parent, tb.n_nodes, an, at, na,
                                                 st.workspace), 1, reps=32), 2)
    ai = W.make_attention_inputs(tb, 1, cfg.num_q_heads, cfg.num_kv_heads, smax, seed=1, device=dev)
    res["copy_us"] = round(graph_us_per_launch(lambda i, f: tb.prefix_len.copy_(p0), 1, reps=32), 2)
    # (kv_commit advances prefix_len: every commit is preceded by the prefix reset)
    res["copy+kv_commit_us"] = round(graph_us_per_launch(
        lambda i, f: (tb.prefix_len.copy_(p0),
                      spi.specinfer_kv_commit(shape, ai.k_cache, ai.v_cache, tb.prefix_len, an, na)), 1, reps=32), 2)
    tb.prefix_len.copy_(p0)
    print(json.dumps(res))


if __name__ == "__main__":
    main()
