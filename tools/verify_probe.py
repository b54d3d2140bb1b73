"""Verify-kernel probe (development tool): device time per launch of verify_greedy / verify_mss /
verify_ns at a config (optionally a batch override), logits cold in L2 as in the bench step (a 256 MB
read-only TMA stream before every launch, as the attention layers before the verifier in the step;
CUDA events around the verify launch only, enqueued behind the flush so the interval is device time).

    python tools/verify_probe.py --config C2 [--batch 2] [--iters 20]
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


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="C2")
    ap.add_argument("--batch", type=int, default=None)
    ap.add_argument("--iters", type=int, default=20)
    ap.add_argument("--lib", default=None, help="A/B: load another build of libspecinfer.so")
    a = ap.parse_args()
    if a.lib:
        spi.load_library(a.lib)
    cfg = W.CONFIGS[a.config]
    if a.batch:
        cfg = dataclasses.replace(cfg, batch=a.batch)
    dev = torch.device("cuda:0")
    tb = W.config_tree_batch(cfg, device=dev)
    B, Lp = cfg.batch, cfg.max_depth + 1
    shape = spi.make_shape(B, tb.max_nodes, 1, 1, cfg.prefix + tb.max_nodes, vocab=cfg.vocab,
                           max_depth=cfg.max_depth)
    st = spi.TreeState.create(shape, tb.parent, tb.depth, tb.prefix_len, tb.n_nodes)
    st.prepare()
    an = torch.empty((B, Lp), dtype=torch.int32, device=dev)
    at, na = torch.empty_like(an), torch.empty((B,), dtype=torch.int32, device=dev)
    flush = torch.zeros(256 << 20, dtype=torch.uint8, device=dev)
    spi.specinfer_hbm_read_probe(flush)   # clean L2 lines: the step reads its logits after a read-only stream
    res = {"config": a.config, "batch": B, "nodes": int(tb.n_nodes.sum().item()), "vocab": cfg.vocab}
    for mode in ("greedy", "mss", "ns"):
        vi = W.make_verify_inputs(tb, cfg.vocab, seed=cfg.seed, mode="mss" if mode == "mss" else "greedy",
                                  device=dev)

        def run():
            if mode == "greedy":
                spi.specinfer_verify_greedy(shape, vi.logits, vi.tree_tokens, tb.parent, tb.n_nodes, an, at, na,
                                            st.workspace)
            elif mode == "mss":
                spi.specinfer_verify_mss(shape, vi.logits, vi.tree_tokens, tb.parent, tb.n_nodes, vi.draft_probs,
                                         1.0, 2, 0, None, an, at, na, st.workspace)
            else:
                spi.specinfer_verify_ns(shape, vi.logits, vi.tree_tokens, tb.parent, tb.n_nodes, 1.0, 2, 0, None,
                                        an, at, na, st.workspace)
        for _ in range(3):
            run()
        torch.cuda.synchronize()
        ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(a.iters)]
        for e0, e1 in ev:
            spi.specinfer_hbm_read_probe(flush)
            e0.record()
            run()
            e1.record()
        torch.cuda.synchronize()
        us = sorted(e0.elapsed_time(e1) * 1e3 for e0, e1 in ev)[a.iters // 2]
        bytes_read = res["nodes"] * cfg.vocab * 4
        res[mode] = {"us": round(us, 2), "logits_GBps": round(bytes_read / us / 1e3, 1)}
    # references on the same bytes: torch's argmax over the logits rows (a library reduction) and the
    # TMA read probe (a pure stream)
    lg = vi.logits
    for name, fn in (("torch_argmax", lambda: torch.argmax(lg, dim=-1)),
                     ("read_probe", lambda: spi.specinfer_hbm_read_probe(lg))):
        for _ in range(3):
            fn()
        ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(a.iters)]
        for e0, e1 in ev:
            spi.specinfer_hbm_read_probe(flush)
            e0.record()
            fn()
            e1.record()
        torch.cuda.synchronize()
        us = sorted(e0.elapsed_time(e1) * 1e3 for e0, e1 in ev)[a.iters // 2]
        res[name] = {"us": round(us, 2), "GBps": round(lg.numel() * 4 / us / 1e3, 1)}
    print(json.dumps(res))


if __name__ == "__main__":
    main()
