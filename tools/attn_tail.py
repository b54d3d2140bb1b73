"""Per-CTA exit times of one tree-attention launch (development tool): which CTAs form the tail.
    python tools/attn_tail.py [--config C2] [--batch 1]"""
import argparse, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import paper_conf_asplos_miaoozcwzwzyssc24_b200 as spi
from paper_conf_asplos_miaoozcwzwzyssc24_b200 import build_lib
import workloads as W

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="C2")
ap.add_argument("--batch", type=int, default=1)
ap.add_argument("--prefix", type=int, default=None)
ap.add_argument("--expansion", default=None, help="override the tree: comma list <k1,..,km>")
ap.add_argument("--flags", type=int, default=0, help="debug flags (64: no split-KV clusters)")
ap.add_argument("--all", action="store_true", help="print every traced tile of CTAs 0-1")
ap.add_argument("--lib", default=None, help="a debug-hooks library built elsewhere (A/B experiments)")
a = ap.parse_args()
spi.load_library(a.lib or build_lib.build(debug_hooks=True))  # traces exist only in the development build
os.environ["SPECINFER_DEBUG_FLAGS"] = str(a.flags)
spi.specinfer_debug_set_trace(None)
cfg = W.CONFIGS[a.config]
dev = torch.device("cuda:0")
P = a.prefix or cfg.prefix
p, d = cfg.tree if not a.expansion else W.expansion_tree([int(x) for x in a.expansion.split(",")])
tb = W.make_tree_batch([(p, d)] * a.batch, [P] * a.batch, device=dev, max_depth=max(cfg.max_depth, int(d.max())))
smax = P + tb.max_nodes
ai = W.make_attention_inputs(tb, 1, cfg.num_q_heads, cfg.num_kv_heads, smax, seed=1, device=dev)
shape = spi.make_shape(a.batch, tb.max_nodes, cfg.num_q_heads, cfg.num_kv_heads, smax, max_depth=tb.max_depth)
st = spi.TreeState.create(shape, tb.parent, tb.depth, tb.prefix_len, tb.n_nodes)
st.prepare()
out = torch.empty_like(ai.q[0])
for _ in range(3):
    st.attention(ai.q[0], ai.k_cache[0], ai.v_cache[0], out)
torch.cuda.synchronize()
tr = torch.zeros(8 * 64 * 16 + 8 * 1024, dtype=torch.int64, device=dev)
spi.specinfer_debug_set_trace(tr)
torch.cuda.synchronize()
st.attention(ai.q[0], ai.k_cache[0], ai.v_cache[0], out)
torch.cuda.synchronize()
spi.specinfer_debug_set_trace(None)
kt = tr.cpu().numpy().astype(np.int64)[8 * 64 * 16:].reshape(-1, 8)[:148]
kt = kt[kt[:, 0] > 0]  # CTAs of this launch (the grid may be smaller than 148)
t0 = kt[:, 0].min()
ex = (kt[:, 1] - t0) / 1e3
fk = np.where(kt[:, 2] > 0, (kt[:, 2] - t0) / 1e3, -1)
order = np.argsort(ex)
names = ["entry", "exit", "first K issue", "cluster barrier", "prologue done", "dependency wait passed",
         "schedule read", "first S ready"]
for k in [0, 4, 5, 6, 2, 7, 3, 1]:
    v = kt[:, k]
    v = v[v > 0]
    if len(v):
        print(f"  {names[k]:24s} us p0/p50/p100: {np.percentile((v - t0) / 1e3, [0, 50, 100]).round(2)}")
print("exit us percentiles 0/25/50/75/90/100:", np.percentile(ex, [0, 25, 50, 75, 90, 100]).round(2))
print("latest 12 CTAs (cta, entry, firstK, exit):")
for c in order[-12:]:
    print(f"  {c:4d} {(kt[c,0]-t0)/1e3:7.2f} {fk[c]:7.2f} {ex[c]:7.2f}")
print("earliest 5:", [(int(c), round(float(ex[c]), 2)) for c in order[:5]])
if a.config in ("C3", "C4"):   # rows kernel: slot 3 holds smid + 1
    sm = kt[:, 3] - 1
    print("exit us by CTA:", " ".join(f"{c}:{ex[c]:.0f}/sm{sm[c]}" for c in range(len(ex))))
if (kt[:, 3] > 0).any():
    s3 = (kt[:, 3] - t0) / 1e3
    print("split-KV: first cluster barrier passed (us) min/median/max:", np.percentile(s3[kt[:, 3] > 0], [0, 50, 100]).round(2))
t = tr.cpu().numpy().astype(np.int64)[:8 * 64 * 16].reshape(8, 64, 16)
for c in range(8):
    x = t[c]
    nv = int((x[:, 0] > 0).sum())
    base = x[0, 0]
    print(f"CTA {c} exit {ex[c]:.2f} us, raw per-tile events (cycles rel. to its first K issue; -1 none): "
          "K-iss V-iss S-mma PV-mma 4..11")
    show = list(range(min(nv + 1, 8))) + [i for i in range(max(8, nv - 3), min(nv + 2, 64))]
    if a.all and c < 2:
        show = list(range(min(nv + 1, 64)))
    for i in show:
        print(f"  {i:3d} " + " ".join(f"{(v - base) if v else -1:7d}" for v in x[i, :16]))
