"""bench.py — SpecInfer token-tree verification hot path on B200.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config C2] [--impl ours|reference]

One step = one verification iteration of the whole hot path over one
batch of synthetic input: tree_prepare -> L x tree_attention -> verify_greedy and/or
verify_mss -> (N>1: NCCL all-gather of accepted tokens) -> kv_commit.  The default workload is
BASELINE.json configs[1] (C2, LLaMA-7B shape), the configuration the metric is quoted on.

Prints ONE JSON line (rank 0).  `value` = verified tree tokens / s for the whole job with
inputs resident in HBM; `e2e` = the same metric through the public API with host buffers
(H2D of the step's q / logits / draft probabilities / tree, D2H of the accepted tokens inside
the timed region).  `roofline` reports the dominant kernel (tree attention) against the
measured HBM copy bandwidth; `cpu_baseline` times the fp64 oracle on a bounded sample.
`--impl reference` times the oracle itself as the reference arm (there is no reference code).
"""
from __future__ import annotations

import argparse
import json
import math
import os
import statistics
import subprocess
import sys
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np
import torch

import workloads as W

METRIC = "verified tree tokens/s/GPU at LLaMA-7B shape; KV-stream GB/s vs HBM peak"
UNIT = "tree tokens/s"


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--config", default="C2", choices=sorted(W.CONFIGS))
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--layers", type=int, default=None, help="override layer count (sweeps only)")
    ap.add_argument("--batch", type=int, default=None, help="override per-GPU batch (sweeps only)")
    ap.add_argument("--prefix", type=int, default=None, help="override prefix (sweeps only)")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--verify", default=None, help="comma list overriding the config's verify modes")
    ap.add_argument("--shard", default="auto", choices=["auto", "request", "kv"],
                    help="N > 1 layout: request sharding, or kv-head sharding (GQA; auto for G > 1)")
    return ap.parse_args()


# ------------------------------------------------------------------------------------------
# distributed plumbing (one process per GPU; torchrun env)
# ------------------------------------------------------------------------------------------
def dist_env():
    ws = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return ws, rank, local


def max_over_ranks(x: float, ws: int, device) -> float:
    if ws == 1:
        return x
    t = torch.tensor([x], dtype=torch.float64, device=device)
    torch.distributed.all_reduce(t, op=torch.distributed.ReduceOp.MAX)
    return float(t.item())


def barrier(ws):
    if ws > 1:
        torch.distributed.barrier()


# ------------------------------------------------------------------------------------------
# clocks sampler (nvidia-smi during the timed region)
# ------------------------------------------------------------------------------------------
class ClockSampler:
    Q = ("clocks.sm,clocks.max.sm,clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, index: int):
        self.index = index
        self.proc = None
        self.path = f"/tmp/specinfer_clocks_{os.getpid()}.csv"

    def start(self):
        try:
            self.f = open(self.path, "w")
            self.proc = subprocess.Popen(["nvidia-smi", f"--query-gpu={self.Q}", "--format=csv,noheader,nounits",
                                          "-i", str(self.index), "-lms", "100"], stdout=self.f,
                                         stderr=subprocess.DEVNULL)
        except Exception:
            self.proc = None

    def stop(self):
        if self.proc is None:
            return None
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except Exception:
            self.proc.kill()
        self.f.close()
        rows = []
        for line in open(self.path):
            parts = [p.strip() for p in line.split(",")]
            if len(parts) != 6:
                continue
            try:
                rows.append((float(parts[0]), float(parts[1]), parts[2:]))
            except ValueError:
                continue
        os.unlink(self.path)
        if not rows:
            return None
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[i] for _, _, r in rows for i, v in enumerate(r) if v.lower() == "active"})
        return {"sm_mhz": statistics.median(r[0] for r in rows), "sm_max_mhz": max(r[1] for r in rows),
                "reasons": reasons, "samples": len(rows)}


# ------------------------------------------------------------------------------------------
# workload
# ------------------------------------------------------------------------------------------
class Workload:
    """One GPU's share of the step.  Request sharding: this rank's B requests end to end.  kv-head
    sharding (GQA, N > 1): attention and KV commit over ALL B*N requests for this rank's Hkv/N
    kv-heads (and their q-heads), verification over this rank's B requests (dist.py)."""

    def __init__(self, cfg: W.Config, args, rank: int, device, ws: int = 1, kv_shard: bool = False):
        self.cfg = cfg
        self.L = args.layers or cfg.layers
        self.B = args.batch or cfg.batch
        self.P = args.prefix or cfg.prefix
        self.kv_shard = kv_shard
        self.Batt = self.B * ws if kv_shard else self.B
        self.Hq, self.Hkv, self.V = cfg.num_q_heads, cfg.num_kv_heads, cfg.vocab
        self.req_lo = rank * self.B if kv_shard else 0
        if kv_shard:
            from paper_conf_asplos_miaoozcwzwzyssc24_b200 import dist as D
            _, self.Hkv, _, self.Hq = D.shard_kv_heads(cfg.num_q_heads, cfg.num_kv_heads, ws, rank)
        self.verify = tuple(args.verify.split(",")) if args.verify else cfg.verify
        parent, depth = cfg.tree
        self.N = int(parent.shape[0])
        self.Dmax = cfg.max_depth
        self.smax = self.P + self.N
        self.device = device
        self.tb = W.make_tree_batch([(parent, depth)] * self.Batt, [self.P] * self.Batt, device=device,
                                    max_depth=self.Dmax)
        seed = cfg.seed + 1000 * rank
        self.ai = W.make_attention_inputs(self.tb, self.L, self.Hq, self.Hkv, self.smax, seed=seed, device=device)
        mode = "mss" if self.verify == ("mss",) else "greedy"
        lo, hi = self.req_lo, self.req_lo + self.B
        self.tbv = W.TreeBatch(self.tb.parent[lo:hi], self.tb.depth[lo:hi], self.tb.prefix_len[lo:hi],
                               self.tb.n_nodes[lo:hi], self.tb.max_nodes, self.tb.max_depth)
        self.vi = W.make_verify_inputs(self.tbv, self.V, seed=seed, mode=mode, device=device)
        self.rids = torch.arange(rank * self.B, (rank + 1) * self.B, dtype=torch.int32, device=device)
        self.bytes_launch = self.attn_bytes_per_launch()   # before any commit moves prefix_len
        self.flops_launch = self.attn_flops_per_launch()

    def tree_tokens_per_step(self) -> int:
        """Tree tokens this rank verifies per step (its B requests)."""
        return int(self.tbv.n_nodes.sum().item())

    def attn_bytes_per_launch(self) -> int:
        """Algorithmic bytes of one tree_attention launch: K and V of every
        (request, kv-head) read once, q read once, out written once."""
        pl = self.tb.prefix_len.cpu().numpy().astype(np.int64)
        n = self.tb.n_nodes.cpu().numpy().astype(np.int64)
        kv = int(((pl + n) * self.Hkv * 128 * 2 * 2).sum())
        qo = int((n * self.Hq * 128 * 2 * 2).sum())
        return kv + qo

    def attn_flops_per_launch(self) -> int:
        pl = self.tb.prefix_len.cpu().numpy().astype(np.int64)
        n = self.tb.n_nodes.cpu().numpy().astype(np.int64)
        dep = self.tb.depth.cpu().numpy()
        tree_pairs = np.array([int((dep[b, :n[b]] + 1).sum()) for b in range(self.Batt)])
        return int((4 * 128 * (n * pl + tree_pairs) * self.Hq).sum())


def run_ours(args, ws, rank, local):
    import paper_conf_asplos_miaoozcwzwzyssc24_b200 as spi

    device = torch.device("cuda", local)
    torch.cuda.set_device(device)
    cfg = W.CONFIGS[args.config]
    G = cfg.num_q_heads // cfg.num_kv_heads
    # (--shard kv also runs at N = 1, where the gather degenerates to a copy: exercises the layout)
    kv_shard = args.shard == "kv" or (ws > 1 and args.shard == "auto" and G > 1 and cfg.num_kv_heads % ws == 0)
    wl = Workload(cfg, args, rank, device, ws=ws, kv_shard=kv_shard)
    L, B, N, Dmax = wl.L, wl.B, wl.N, wl.Dmax
    Ba = wl.Batt
    Lp = Dmax + 1
    # attention / commit shape (all B*N requests x local heads when kv-sharded) and verify shape
    shape = spi.make_shape(Ba, N, wl.Hq, wl.Hkv, wl.smax, num_layers=L, vocab=wl.V, max_depth=Dmax)
    st = spi.TreeState.create(shape, wl.tb.parent, wl.tb.depth, wl.tb.prefix_len, wl.tb.n_nodes)
    if kv_shard:
        shape_v = spi.make_shape(B, N, 1, 1, wl.smax, num_layers=L, vocab=wl.V, max_depth=Dmax)
        st_v = spi.TreeState.create(shape_v, wl.tbv.parent, wl.tbv.depth, wl.tbv.prefix_len, wl.tbv.n_nodes)
    else:
        shape_v, st_v = shape, st
    out = torch.empty_like(wl.ai.q)
    prefix0 = wl.tb.prefix_len.clone()
    an = torch.empty((B, Lp), dtype=torch.int32, device=device)
    at, na = torch.empty_like(an), torch.empty((B,), dtype=torch.int32, device=device)
    an2, at2, na2 = torch.empty_like(an), torch.empty_like(an), torch.empty_like(na)
    gather_in = torch.empty((B, 2 * Lp + 1), dtype=torch.int32, device=device)
    gather_out = torch.empty((ws * B, 2 * Lp + 1), dtype=torch.int32, device=device)
    an_all = torch.empty((Ba, Lp), dtype=torch.int32, device=device)   # kv-sharded commit input
    na_all = torch.empty((Ba,), dtype=torch.int32, device=device)
    iteration = [0]

    def seg_prepare():
        wl.tb.prefix_len.copy_(prefix0)
        st.prepare()
        if kv_shard:
            st_v.prepare()

    def seg_attention():
        for l in range(L):
            st.attention(wl.ai.q[l], wl.ai.k_cache[l], wl.ai.v_cache[l], out[l])

    def seg_verify():
        if "greedy" in wl.verify:
            spi.specinfer_verify_greedy(shape_v, wl.vi.logits, wl.vi.tree_tokens, wl.tbv.parent, wl.tbv.n_nodes,
                                        an, at, na, st_v.workspace)
        if "mss" in wl.verify:
            spi.specinfer_verify_mss(shape_v, wl.vi.logits, wl.vi.tree_tokens, wl.tbv.parent, wl.tbv.n_nodes,
                                     wl.vi.draft_probs, 1.0, cfg.seed, 0, wl.rids, an2, at2, na2, st_v.workspace)

    def seg_commit():
        if kv_shard:
            # every request's accepted path (gathered) -> this rank's kv-head shard of its cache
            n_all, _, nodes_all = D.unpack_accepted(gather_out)
            na_all.copy_(n_all)
            an_all.copy_(nodes_all)
            src = (an_all, na_all)
        else:
            src = (an, na) if "greedy" in wl.verify else (an2, na2)
        spi.specinfer_kv_commit(shape, wl.ai.k_cache, wl.ai.v_cache, wl.tb.prefix_len, src[0], src[1])

    launches_per_step = (spi.specinfer_launches_per_call("tree_prepare") * (2 if kv_shard else 1) +
                         L * spi.specinfer_launches_per_call("tree_attention") +
                         ("greedy" in wl.verify) * spi.specinfer_launches_per_call("verify_greedy") +
                         ("mss" in wl.verify) * spi.specinfer_launches_per_call("verify_mss") +
                         spi.specinfer_launches_per_call("kv_commit"))

    from paper_conf_asplos_miaoozcwzwzyssc24_b200 import dist as D

    def gather():
        # a7: the tokens-only exchange after verification, NCCL over NVLink
        if ws > 1 or kv_shard:
            src = (na, at, an) if "greedy" in wl.verify else (na2, at2, an2)
            gather_in.copy_(D.pack_accepted(*src))
            if ws > 1:
                D.gather_accepted(gather_in, gather_out)
            else:
                gather_out.copy_(gather_in)

    def seg_verify_commit():
        seg_verify()
        gather()
        seg_commit()

    # ---- capture the segments as CUDA graphs (one launch each per step; the gather stays eager) ----
    s = torch.cuda.Stream(device)
    s.wait_stream(torch.cuda.current_stream(device))
    with torch.cuda.stream(s):
        for _ in range(2):  # eager warm-up (lazy init, tensor-map encode, func attributes)
            seg_prepare(); seg_attention(); seg_verify_commit()
    torch.cuda.synchronize(device)
    graphs = []
    for fn in (seg_prepare, seg_attention, seg_verify, seg_commit):
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g, stream=s):
            fn()
        graphs.append(g)
    torch.cuda.synchronize(device)

    def step():
        graphs[0].replay()
        graphs[1].replay()
        graphs[2].replay()
        gather()
        graphs[3].replay()

    with torch.cuda.stream(s):
        for _ in range(args.warmup):
            step()
    torch.cuda.synchronize(device)
    K = args.steps
    ev = [torch.cuda.Event(enable_timing=True) for _ in range(2 * K + 2)]
    sampler = ClockSampler(local) if rank == 0 else None
    barrier(ws)
    torch.cuda.synchronize(device)
    if sampler:
        sampler.start()
        time.sleep(0.3)
    with torch.cuda.stream(s):
        ev[0].record(s)
        for k in range(K):
            graphs[0].replay()
            ev[2 + 2 * k].record(s)
            graphs[1].replay()
            ev[3 + 2 * k].record(s)
            graphs[2].replay()
            gather()
            graphs[3].replay()
        ev[1].record(s)
    torch.cuda.synchronize(device)
    barrier(ws)
    clocks = sampler.stop() if sampler else None
    total_ms = ev[0].elapsed_time(ev[1])
    attn_ms = sum(ev[2 + 2 * k].elapsed_time(ev[3 + 2 * k]) for k in range(K))
    total_ms = max_over_ranks(total_ms, ws, device)
    attn_ms_max = max_over_ranks(attn_ms, ws, device)
    ms_per_step = total_ms / K
    tokens_step = wl.tree_tokens_per_step()
    value = tokens_step * ws * K / (total_ms / 1e3)
    acc_mean = float((na if "greedy" in wl.verify else na2).float().mean().item())
    acc_mss = float(na2.float().mean().item()) if "mss" in wl.verify else None

    # ---- roofline of the dominant kernel (tree attention), measured in the timed region ----
    attn_launch_s = attn_ms_max / (K * L) / 1e3
    bytes_launch = wl.bytes_launch
    flops_launch = wl.flops_launch
    peaks = {}
    try:
        peaks = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
        peak, peak_src = float(peaks["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    except Exception:
        peak, peak_src = 6650.0, "fallback (B200_PROFILING.md)"
    achieved = bytes_launch / attn_launch_s / 1e9
    traffic = None
    try:
        tr = json.load(open(os.path.join(ROOT, "profiles", "ncu_traffic.json")))
        ent = tr.get(f"{args.config}:L{L}:B{B}:P{wl.P}") or tr.get(args.config)
        if ent:
            traffic = ent["dram_bytes_per_launch"]
    except Exception:
        pass
    # a kernel timed inside a long step takes the sustained tensor figure when the driver measured it
    tf_peak, tf_src = 1590.0, "fallback (B200_PROFILING.md)"
    if peaks:
        if "bf16_tflops_sustained" in peaks:
            tf_peak, tf_src = float(peaks["bf16_tflops_sustained"]), "measured sustained (MEASURED_PEAKS.json)"
        elif "bf16_tflops" in peaks:
            tf_peak, tf_src = float(peaks["bf16_tflops"]), "measured burst (MEASURED_PEAKS.json)"
    rows_per_kv_head = (wl.Hq // wl.Hkv) * wl.tb.max_nodes
    kname = "tree_attn_rows_kernel" if rows_per_kv_head > 64 else "tree_attn_kernel"
    tflops = flops_launch / attn_launch_s / 1e12
    ai_launch = flops_launch / bytes_launch
    ridge = tf_peak * 1e3 / peak  # flop per byte where the two roofs meet
    if ai_launch > ridge:
        roofline = {"bound": "tensor", "kernel": kname, "achieved": round(tflops, 2), "peak": tf_peak,
                    "unit": "TFLOP/s", "frac": round(tflops / tf_peak, 4), "traffic": traffic,
                    "peak_source": tf_src, "algorithmic_flops_per_launch": flops_launch,
                    "hbm_gbs": round(achieved, 1), "hbm_frac": round(achieved / peak, 4), "hbm_peak": peak,
                    "hbm_peak_source": peak_src}
    else:
        roofline = {"bound": "hbm", "kernel": kname, "achieved": round(achieved, 1), "peak": peak,
                    "unit": "GB/s", "frac": round(achieved / peak, 4), "traffic": traffic,
                    "peak_source": peak_src, "tensor_tflops": round(tflops, 2),
                    "tensor_frac": round(tflops / tf_peak, 4), "tensor_peak": tf_peak}
    # BASELINE.json's north star quotes the KV stream against "about 8 TB/s": context only
    roofline["hbm_frac_of_8TBps"] = round(achieved / 8000.0, 4)
    roofline.update({"algorithmic_bytes_per_launch": bytes_launch, "arithmetic_intensity": round(ai_launch, 1),
                     "avg_launch_us": round(attn_launch_s * 1e6, 2),
                     "share_of_step": round(attn_ms_max / total_ms, 4)})

    # ---- end to end through the public API with host buffers ----
    e2e = None
    if not args.no_e2e:
        h_q = torch.empty_like(wl.ai.q, device="cpu").pin_memory()
        h_q.copy_(wl.ai.q)
        h_logits = wl.vi.logits.cpu().pin_memory()
        h_draft = wl.vi.draft_probs.cpu().pin_memory() if "mss" in wl.verify else None
        h_tree = [t.cpu().pin_memory() for t in (wl.tb.parent, wl.tb.depth, wl.vi.tree_tokens, wl.tb.n_nodes, prefix0)]
        h_res_a = torch.empty((B, Lp), dtype=torch.int32).pin_memory()
        h_res_n = torch.empty((B,), dtype=torch.int32).pin_memory()
        res_a, res_n = (at, na) if "greedy" in wl.verify else (at2, na2)
        dsts = [wl.tb.parent, wl.tb.depth, wl.vi.tree_tokens, wl.tb.n_nodes, prefix0]
        h2d = h_q.numel() * 2 + h_logits.numel() * 4 + (h_draft.numel() * 4 if h_draft is not None else 0) + \
            sum(t.numel() * 4 for t in h_tree)
        d2h = h_res_a.numel() * 4 + h_res_n.numel() * 4

        # One CUDA graph per step: the H2D copies run on a copy stream (pinned memory, the copy
        # engines) and each layer's attention waits only for its own q, so the PCIe transfer of
        # layer l+1's q and of the logits / draft probabilities overlaps the attention of layer l.
        copy_s = torch.cuda.Stream(device)
        ev_fork = torch.cuda.Event()
        ev_tree = torch.cuda.Event()
        ev_q = [torch.cuda.Event() for _ in range(L)]
        ev_lg = torch.cuda.Event()

        def e2e_step():
            ev_fork.record(s)
            copy_s.wait_event(ev_fork)
            with torch.cuda.stream(copy_s):
                for d, h in zip(dsts, h_tree):
                    d.copy_(h, non_blocking=True)
                ev_tree.record(copy_s)
                for l in range(L):
                    wl.ai.q[l].copy_(h_q[l], non_blocking=True)
                    ev_q[l].record(copy_s)
                wl.vi.logits.copy_(h_logits, non_blocking=True)
                if h_draft is not None:
                    wl.vi.draft_probs.copy_(h_draft, non_blocking=True)
                ev_lg.record(copy_s)
            s.wait_event(ev_tree)
            seg_prepare()
            for l in range(L):
                s.wait_event(ev_q[l])
                st.attention(wl.ai.q[l], wl.ai.k_cache[l], wl.ai.v_cache[l], out[l])
            s.wait_event(ev_lg)
            seg_verify_commit()
            h_res_a.copy_(res_a, non_blocking=True)
            h_res_n.copy_(res_n, non_blocking=True)

        with torch.cuda.stream(s):
            e2e_step()  # eager warm-up of the multi-stream step
        torch.cuda.synchronize(device)
        g_e2e = None
        if ws == 1:
            g_e2e = torch.cuda.CUDAGraph()
            with torch.cuda.graph(g_e2e, stream=s):
                e2e_step()
            torch.cuda.synchronize(device)

        def e2e_run():
            if g_e2e is not None:
                g_e2e.replay()
            else:
                e2e_step()

        with torch.cuda.stream(s):
            for _ in range(max(1, args.warmup // 2)):
                e2e_run()
        torch.cuda.synchronize(device)
        barrier(ws)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        with torch.cuda.stream(s):
            e0.record(s)
            for _ in range(K):
                e2e_run()
            e1.record(s)
        torch.cuda.synchronize(device)
        barrier(ws)
        e2e_ms = max_over_ranks(e0.elapsed_time(e1), ws, device)
        e2e = {"value": round(tokens_step * ws * K / (e2e_ms / 1e3), 1), "unit": UNIT,
               "h2d_bytes_per_step": int(h2d), "d2h_bytes_per_step": int(d2h),
               "ms_per_step": round(e2e_ms / K, 4),
               "inputs": "per step from pinned host memory: tree arrays, q of every layer, logits"
                         + (", draft probabilities" if h_draft is not None else "")
                         + "; result read back: accepted tokens + counts; H2D on a copy stream "
                           "overlapping the attention of earlier layers"}

    cpu = None
    if rank == 0 and ws == 1 and not args.no_cpu:
        wl.tb.prefix_len.copy_(prefix0)   # undo the last step's commit: the sample is a fresh iteration
        torch.cuda.synchronize(device)
        cpu = cpu_baseline(wl)

    line = {
        "metric": METRIC, "value": round(value, 1), "unit": UNIT, "n_gpus": ws, "steps": K,
        "warmup": args.warmup, "ms_per_step": round(ms_per_step, 4), "higher_is_better": True,
        "scaling": "weak", "vs_baseline": None, "dtype": "bf16", "data": "synthetic",
        "config": {"workload": f"{cfg.name}: {cfg.description}", "layers": L, "batch_per_gpu": B,
                   "global_batch": B * ws, "prefix": wl.P, "tree_nodes": N, "max_depth": Dmax,
                   "num_q_heads": wl.Hq, "num_kv_heads": wl.Hkv, "vocab": wl.V, "verify": list(wl.verify),
                   "parallelism": (f"kv-head-sharded attention/commit x{ws}, request-sharded verification" if kv_shard
                                   else f"request-sharded x{ws}") if ws > 1 else "single GPU",
                   "l2": "no flush: every step streams the full KV cache "
                         f"({2 * L * B * wl.Hkv * wl.smax * 256 / 1e9:.1f} GB/GPU) >> 126 MB L2",
                   "graph": "4 CUDA graphs per step (prepare | L x attention | verify | commit), NCCL gather between"},
        "roofline": roofline, "cpu_baseline": cpu, "e2e": e2e,
        "gpu_launches": launches_per_step * K, "clocks": clocks,
        "extra": {"tree_tokens_per_step": tokens_step * ws, "mean_n_accepted_greedy": acc_mean if "greedy" in wl.verify else None,
                  "mean_n_accepted_mss": acc_mss,
                  "accepted_tokens_per_s": round(float((na if "greedy" in wl.verify else na2).sum().item()) * ws * K /
                                                 (total_ms / 1e3), 1),
                  "attention_ms_per_step": round(attn_ms_max / K, 4)},
    }
    if rank == 0:
        print(json.dumps(line), flush=True)


# ------------------------------------------------------------------------------------------
# CPU baseline: the fp64 oracle as it stands, on a bounded sample of the same workload
# ------------------------------------------------------------------------------------------
def _oracle_sample(wl: Workload, n_req: int, layers=(0,)):
    """Times the fp64 oracle (as it stands) on `n_req` requests of the workload: tree attention of the
    given layers, then greedy / MSS verification of those requests."""
    import oracle
    cores = len(os.sched_getaffinity(0))
    os.environ["OMP_NUM_THREADS"] = str(cores)
    tb = wl.tb
    par, dep = tb.parent[:n_req].cpu(), tb.depth[:n_req].cpu()
    pl, nn_ = tb.prefix_len[:n_req].cpu(), tb.n_nodes[:n_req].cpu()
    lg = wl.vi.logits[:n_req].cpu().numpy()
    toks = wl.vi.tree_tokens[:n_req].cpu().numpy()
    dr = wl.vi.draft_probs[:n_req].cpu().numpy() if "mss" in wl.verify else None
    ta = 0.0
    for l in layers:
        q = wl.ai.q[l, :n_req].cpu()
        k = wl.ai.k_cache[l, :n_req].cpu()
        v = wl.ai.v_cache[l, :n_req].cpu()
        t0 = time.perf_counter()
        oracle.tree_attention(q, k, v, par, dep, pl, nn_)
        ta += time.perf_counter() - t0
    t1 = time.perf_counter()
    if "greedy" in wl.verify:
        oracle.verify_greedy(lg, toks, par.numpy(), nn_.numpy(), path_len=wl.Dmax + 1)
    if "mss" in wl.verify:
        oracle.verify_mss(lg, toks, par.numpy(), nn_.numpy(), dr, seed=1, path_len=wl.Dmax + 1)
    tv = time.perf_counter() - t1
    return ta, tv, cores


def cpu_baseline(wl: Workload, budget_s: float = 12.0):
    """The oracle timed on the host cores on a bounded sample (~10-20 s): every request of the
    step, as many layers as fit the budget (extrapolated linearly to all layers when fewer)."""
    import oracle  # noqa: F401  (test infrastructure; only this leg and --impl reference use it)
    ta1, tv, cores = _oracle_sample(wl, wl.B, layers=(0,))
    n_layers = int(max(1, min(wl.L, budget_s // max(ta1, 1e-3))))
    if n_layers > 1:
        ta, tv, cores = _oracle_sample(wl, wl.B, layers=tuple(range(n_layers)))
    else:
        ta = ta1
    t_step = ta * wl.L / n_layers + tv
    tokens = wl.tree_tokens_per_step()
    extra = "" if n_layers == wl.L else f", x{wl.L / n_layers:.1f} extrapolated to {wl.L} layers"
    return {"value": round(tokens / t_step, 3), "unit": UNIT, "cores": cores, "kind": "oracle",
            "sample": f"all {wl.B} requests, tree attention of {n_layers} of {wl.L} layers "
                      f"({ta:.1f} s fp64{extra}) + greedy/MSS verification ({tv:.2f} s)"}


def run_reference(args, ws, rank, local):
    """Reference arm: the oracle timed on the host cores (there is no reference code; PAPER.md
    only).  Rank 0 alone runs at N>1."""
    if rank != 0:
        return
    cfg = W.CONFIGS[args.config]
    device = torch.device("cuda", local) if torch.cuda.is_available() else torch.device("cpu")
    a = argparse.Namespace(**vars(args))
    a.batch = 1
    wl = Workload(cfg, a, 0, device)
    for _ in range(args.warmup):
        _oracle_sample(wl, 1)
    t_tot = 0.0
    tokens = 0
    cores = 1
    for it in range(args.steps):
        ta, tv, cores = _oracle_sample(wl, 1, layers=(it % wl.L,))
        t_tot += ta * wl.L + tv
        tokens += int(wl.tb.n_nodes[:1].sum().item())
    value = tokens / t_tot
    sample = f"1 request x 1 layer of {cfg.name} tree attention per step (fp64 oracle, x{wl.L} layers extrapolated) + its verification"
    print(json.dumps({
        "impl": "reference", "metric": METRIC, "value": round(value, 3), "unit": UNIT, "n_gpus": ws,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(1e3 * t_tot / args.steps, 3),
        "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
        "config": {"workload": f"{cfg.name}: {cfg.description}"},
        "cpu_baseline": {"value": round(value, 3), "unit": UNIT, "cores": cores, "kind": "oracle", "sample": sample},
        "e2e": {"value": round(value, 3), "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }), flush=True)


def main():
    args = parse()
    ws, rank, local = dist_env()
    if ws != args.gpus and rank == 0:
        print(f"warning: --gpus {args.gpus} but WORLD_SIZE {ws}", file=sys.stderr)
    if ws > 1:
        backend = "nccl" if args.impl == "ours" else "gloo"
        if backend == "nccl":
            torch.cuda.set_device(local)
        torch.distributed.init_process_group(backend)
    try:
        if args.impl == "reference":
            run_reference(args, ws, rank, local)
        else:
            run_ours(args, ws, rank, local)
    finally:
        if ws > 1:
            torch.distributed.destroy_process_group()


if __name__ == "__main__":
    main()
