"""Formats gpurun_out/c5_sweep.jsonl (tools/c5_sweep.py) into profiles/c5_sweep_<round>.md (+ .jsonl copy).
    python tools/c5_report.py r01"""
import json
import os
import shutil
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
R = sys.argv[1] if len(sys.argv) > 1 else "r01"
src = os.path.join(ROOT, "gpurun_out", f"c5_sweep_{R}.jsonl")
if not os.path.exists(src):
    src = os.path.join(ROOT, "gpurun_out", "c5_sweep.jsonl")
rows = [json.loads(l) for l in open(src)]
pk = rows[0]["peaks"]
out = [f"# C5 sweep, round {R[1:]} (`tools/c5_sweep.py`, one B200)", "",
       "BASELINE.json configs[4]: tree size x batch x prefix, LLaMA-7B attention shape (32 heads x 128, MHA), one layer per point,",
       "random trees of exactly n nodes (depth <= 8, fanout <= 8, seeded), greedy verification over V = 32000. Attention: device",
       "time per launch from a CUDA graph of consecutive launches (SPECINFER_ATTN_EARLY_PREFIX after the first, as bench.py runs",
       "the layers) rotating over enough layers' caches that each replay streams > 512 MB (no L2 flush needed; `graph_layers`),",
       "median of 3 replays; verification: CUDA events per launch after a 256 MB L2 flush. Algorithmic bytes per (request,",
       "kv-head) = (P + n)*512 + G*n*512; FLOPs per",
       "(request, q-head) = 4*128*(n*P + sum(depth+1)); bound = the roof the arithmetic intensity hits first",
       f"(ridge = {pk['bf16_tflops'] * 1e3 / pk['hbm_gbs']:.0f} flop/B). Peaks: {pk['hbm_gbs']} GB/s HBM, {pk['bf16_tflops']} TFLOP/s bf16 "
       f"({pk['source']}{', B200_PROFILING.md; MEASURED_PEAKS.json was absent' if pk['source'] == 'fallback' else ''}).",
       "n <= 64 runs the swapped kernel (`tree_attn_kernel<NT>`), n >= 128 the rows-as-M kernel (`tree_attn_rows_kernel`).", "",
       "| n | B | P | attn us | GB/s | HBM frac | TFLOP/s | tensor frac | AI | bound | roofline frac | verify_greedy us | verify GB/s |",
       "|---|---|---|---|---|---|---|---|---|---|---|---|---|"]
for r in rows:
    out.append(f"| {r['n']} | {r['batch']} | {r['prefix']} | {r['attn_us']} | {r['attn_GBps']} | {r['hbm_frac']:.3f} | "
               f"{r['attn_TFps']} | {r['tensor_frac']:.3f} | {r['AI']} | {r['bound']} | {r['roofline_frac']:.3f} | "
               f"{r['verify_greedy_us']} | {r['verify_GBps']} |")
big = [r for r in rows if r['bound'] == 'hbm' and r['n'] <= 64 and r['batch'] * r['prefix'] >= 8 * 8192]
out += ["", f"Memory-bound points with n <= 64 and B*P >= 65536 (>= 1.07 GB of KV per launch): HBM fraction "
        f"{min(r['hbm_frac'] for r in big):.3f}-{max(r['hbm_frac'] for r in big):.3f}.",
        "Fractions slightly above 1 are possible: the denominator is a read+write copy, these launches only read (the TMA",
        "read probe reaches ~6.1-7.0 TB/s on large buffers, `bench.py` roofline). Small points (B = 1, B*P <= 4096) are",
        "latency-bound: a launch covers a few MB and the kernel-boundary costs dominate (dispatch, prologue, first loads,",
        "split merge: `profiles/small_batch_r02.md`). n = 128 / 256 run the rows kernel, bound by its per-tile softmax",
        "instruction stream (`profiles/rows_kernel_r02.md`)."]
open(os.path.join(ROOT, "profiles", f"c5_sweep_{R}.md"), "w").write("\n".join(out) + "\n")
shutil.copy(src, os.path.join(ROOT, "profiles", f"c5_sweep_{R}.jsonl"))
print("\n".join(out[-5:]))
