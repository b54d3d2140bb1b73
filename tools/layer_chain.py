"""Per-CTA timeline of consecutive tree-attention layers inside one CUDA graph (development tool,
needs the debug-hooks build): entry / first K load / cluster barrier / exit of every CTA of every
layer on the global timer, to see how much of a layer's time is prologue, streaming, merge and the
hand-off to the next layer (PDL).

    python tools/layer_chain.py [--config C2] [--batch 2] [--layers 6]
"""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import paper_conf_asplos_miaoozcwzwzyssc24_b200 as spi
import workloads as W
from paper_conf_asplos_miaoozcwzwzyssc24_b200 import build_lib

spi.load_library(build_lib.build(debug_hooks=True))

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="C2")
ap.add_argument("--batch", type=int, default=2)
ap.add_argument("--prefix", type=int, default=None)
ap.add_argument("--layers", type=int, default=6)
ap.add_argument("--flags", type=int, default=0, help="debug flags (64: no split-KV clusters)")
ap.add_argument("--early", action="store_true", help="SPECINFER_ATTN_EARLY_PREFIX on layers >= 1")
a = ap.parse_args()
os.environ["SPECINFER_DEBUG_FLAGS"] = str(a.flags)
spi.specinfer_debug_set_trace(None)
cfg = W.CONFIGS[a.config]
dev = torch.device("cuda:0")
P = a.prefix or cfg.prefix
p, d = cfg.tree
tb = W.make_tree_batch([(p, d)] * a.batch, [P] * a.batch, device=dev, max_depth=cfg.max_depth)
smax = P + tb.max_nodes
L = a.layers
ai = W.make_attention_inputs(tb, L, cfg.num_q_heads, cfg.num_kv_heads, smax, seed=1, device=dev)
shape = spi.make_shape(a.batch, tb.max_nodes, cfg.num_q_heads, cfg.num_kv_heads, smax, max_depth=cfg.max_depth)
st = spi.TreeState.create(shape, tb.parent, tb.depth, tb.prefix_len, tb.n_nodes)
out = torch.empty_like(ai.q)
NTR = 8 * 64 * 16 + 8 * 1024
traces = [torch.zeros(NTR, dtype=torch.int64, device=dev) for _ in range(L)]
s = torch.cuda.Stream(dev)
with torch.cuda.stream(s):
    st.prepare()
    for l in range(L):
        st.attention(ai.q[l], ai.k_cache[l], ai.v_cache[l], out[l])
torch.cuda.synchronize()
g = torch.cuda.CUDAGraph()
with torch.cuda.graph(g, stream=s):
    st.prepare()
    for l in range(L):
        spi.specinfer_debug_set_trace(traces[l])   # baked into this layer's captured launch
        st.attention(ai.q[l], ai.k_cache[l], ai.v_cache[l], out[l], prefetch=a.early and l > 0)
spi.specinfer_debug_set_trace(None)
for _ in range(3):
    g.replay()
torch.cuda.synchronize()
for t in traces:
    t.zero_()
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
with torch.cuda.stream(s):
    e0.record(s)
    g.replay()
    e1.record(s)
torch.cuda.synchronize()
print(f"graph: prepare + {L} layers = {e0.elapsed_time(e1) * 1e3:.1f} us")
kts = [t.cpu().numpy()[8 * 64 * 16:].reshape(-1, 8)[:148] for t in traces]
t0 = min(int(k[k[:, 0] > 0, 0].min()) for k in kts)
print("layer | CTAs | entry min/med/max | firstK min/med/max | barrier med | exit min/med/max (us from first entry)")
prev_exit = None
for l, k in enumerate(kts):
    k = k[k[:, 0] > 0]
    e = (k[:, 0] - t0) / 1e3
    x = (k[:, 1] - t0) / 1e3
    f = (k[k[:, 2] > 0, 2] - t0) / 1e3
    b3 = (k[k[:, 3] > 0, 3] - t0) / 1e3
    q = lambda v: "/".join(f"{y:7.2f}" for y in np.percentile(v, [0, 50, 100])) if len(v) else "-"
    print(f"{l:5d} | {len(k):4d} | {q(e)} | {q(f)} | {np.median(b3) if len(b3) else float('nan'):7.2f} | {q(x)}")
    if prev_exit is not None:
        print(f"      gap: last exit of layer {l-1} -> median first K of layer {l}: {np.median(f) - prev_exit:.2f} us; "
              f"layer span (max exit - prev max exit) {x.max() - prev_exit:.2f} us")
    prev_exit = x.max()
    rel = lambda j: np.median((k[k[:, j] > 0, j] - k[k[:, j] > 0, 0]) / 1e3) if (k[:, j] > 0).any() else float("nan")
    print(f"      per-CTA medians from entry: prologue {rel(4):.2f}, dep-wait {rel(5):.2f}, schedule {rel(6):.2f}, "
          f"first K {rel(2):.2f}, first S ready {rel(7):.2f}, exit {rel(1):.2f} us")
