"""MSS verify probe: per-launch time and (with --trace) the walk timeline of requests 0-15."""
import argparse, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import paper_conf_asplos_miaoozcwzwzyssc24_b200 as spi
from paper_conf_asplos_miaoozcwzwzyssc24_b200 import build_lib
spi.load_library(build_lib.build(debug_hooks=True))  # traces exist only in the development build
import workloads as W

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="C2")
ap.add_argument("--mode", default="greedy")
a = ap.parse_args()
cfg = W.CONFIGS[a.config]
dev = torch.device("cuda:0")
tb = W.config_tree_batch(cfg, device=dev)
shape = spi.make_shape(cfg.batch, tb.max_nodes, 1, 1, cfg.prefix + tb.max_nodes, vocab=cfg.vocab, max_depth=cfg.max_depth)
st = spi.TreeState.create(shape, tb.parent, tb.depth, tb.prefix_len, tb.n_nodes)
st.prepare()
vi = W.make_verify_inputs(tb, cfg.vocab, seed=cfg.seed, mode=a.mode, device=dev)
B, Lp = cfg.batch, cfg.max_depth + 1
an = torch.empty((B, Lp), dtype=torch.int32, device=dev); at = torch.empty_like(an); na = torch.empty((B,), dtype=torch.int32, device=dev)
def run():
    spi.specinfer_verify_mss(shape, vi.logits, vi.tree_tokens, tb.parent, tb.n_nodes, vi.draft_probs, 1.0, 2, 0, None, an, at, na, st.workspace)
for _ in range(3): run()
torch.cuda.synchronize()
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record()
for _ in range(20): run()
e1.record(); torch.cuda.synchronize()
print(f"verify_mss {a.config}: {e0.elapsed_time(e1)*1e3/20:.1f} us/launch; n_accepted {na.tolist()}")
os.environ["SPECINFER_TRACE_MSS"] = "1"
tr = torch.zeros(16 * 64, dtype=torch.int64, device=dev)
spi.specinfer_debug_set_trace(tr)
run(); torch.cuda.synchronize()
os.environ.pop("SPECINFER_TRACE_MSS"); spi.specinfer_debug_set_trace(None)
t = tr.cpu().numpy().reshape(16, 64)
t0 = t[:, 0][t[:, 0] > 0].min()
for b in range(min(B, 16)):
    ev = [(i, (t[b, i] - t0) / 1e3) for i in range(64) if t[b, i] > 0]
    print(b, " ".join(f"{i}:{v:.1f}" for i, v in ev))
