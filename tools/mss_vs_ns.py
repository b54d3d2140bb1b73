"""MSS vs naive sampling on synthetic distributions (the structure of PAPER.md Table 3,
and Theorem 4.3): average tokens verified per stochastic decoding step by
specinfer_verify_mss and specinfer_verify_ns on the same token trees, on the GPU.

Synthetic workload: LLM logits 3 z, draft q = softmax(l + tau eps), children of a
node drawn i.i.d. from its q (the setting of Theorem 4.2, reading R13); trees <1,1,k,1,1,1,1,1>
(the paper's width k, L1078-1079), V = 32000, `--requests` requests per point, several seeds.

    python tools/mss_vs_ns.py [--widths 1,2,3,4,5] [--requests 512] [--seeds 4]
"""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch

import paper_conf_asplos_miaoozcwzwzyssc24_b200 as spi
import workloads as W


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--widths", default="1,2,3,4,5")
    ap.add_argument("--requests", type=int, default=512)
    ap.add_argument("--seeds", type=int, default=4)
    ap.add_argument("--vocab", type=int, default=32000)
    ap.add_argument("--tau", type=float, default=None)
    ap.add_argument("--out", default=None)
    a = ap.parse_args()
    dev = torch.device("cuda:0")
    rows = []
    for k in [int(x) for x in a.widths.split(",")]:
        exp = (1, 1, k, 1, 1, 1, 1, 1)
        par, dep = W.expansion_tree(exp)
        B = a.requests
        tot = {"mss": 0.0, "ns": 0.0}
        cnt = 0
        for s in range(a.seeds):
            tb = W.make_tree_batch([(par, dep)] * B, [0] * B, device=dev, max_depth=len(exp))
            vi = W.make_verify_inputs(tb, a.vocab, seed=1000 * k + s, mode="mss", device=dev, tau=a.tau)
            shape = spi.make_shape(B, tb.max_nodes, 1, 1, tb.max_nodes, vocab=a.vocab, max_depth=len(exp))
            st = spi.TreeState.create(shape, tb.parent, tb.depth, tb.prefix_len, tb.n_nodes)
            st.prepare()
            outs = [torch.empty((B, len(exp) + 1), dtype=torch.int32, device=dev) for _ in range(2)] + \
                   [torch.empty((B,), dtype=torch.int32, device=dev)]
            rids = torch.arange(s * B, (s + 1) * B, dtype=torch.int32, device=dev)
            spi.specinfer_verify_mss(shape, vi.logits, vi.tree_tokens, tb.parent, tb.n_nodes, vi.draft_probs, 1.0,
                                     77, s, rids, *outs, st.workspace)
            tot["mss"] += float(outs[2].float().sum())
            spi.specinfer_verify_ns(shape, vi.logits, vi.tree_tokens, tb.parent, tb.n_nodes, 1.0, 78, s, rids, *outs,
                                    st.workspace)
            tot["ns"] += float(outs[2].float().sum())
            cnt += B
            del vi
            torch.cuda.empty_cache()
        row = {"width": k, "expansion": list(exp), "requests": cnt, "vocab": a.vocab,
               "tokens_per_step": {"naive_sampling": round(tot["ns"] / cnt, 4),
                                   "multi_step_speculative_sampling": round(tot["mss"] / cnt, 4)},
               "improvement": round(tot["mss"] / tot["ns"], 4)}
        print(json.dumps(row), flush=True)
        rows.append(row)
    if a.out:
        with open(a.out, "w") as f:
            for r in rows:
                f.write(json.dumps(r) + "\n")


if __name__ == "__main__":
    main()
