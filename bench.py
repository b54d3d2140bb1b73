"""bench.py — SpecInfer token-tree verification hot path on B200.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config C2] [--scaling strong|weak]
                    [--impl ours|reference]

One step = one verification iteration of the whole hot path over one batch
of synthetic input: tree_prepare -> L x tree_attention -> verify_greedy and/or verify_mss ->
tokens-only gather of the accepted paths (NCCL at N > 1) -> kv_commit
(paper_conf_asplos_miaoozcwzwzyssc24_b200/step.py).  The default workload is BASELINE.json
configs[1] (C2, LLaMA-7B shape), the configuration the metric is quoted on.

Scaling: `strong` (default) keeps the config's GLOBAL batch and splits it over the
N ranks (request sharding; kv-head sharding for GQA configs); `weak` gives every rank the config's
batch.  Every request's inputs come from its own seeded generator, so a rank materialises exactly
its share of the global problem and the integer results equal the N = 1 run's.

Prints ONE JSON line (rank 0).  `value` = verified tree tokens / s for the whole job with inputs
resident in HBM; `e2e` = the same metric through the public API with host buffers (H2D of the
step's q / logits / draft probabilities / tree, D2H of the accepted tokens inside the timed
region).  `roofline` reports the dominant kernel (tree attention) against the measured HBM copy
bandwidth (and the library's TMA read probe on the same bytes); `cpu_baseline` times the fp64
oracle on a bounded sample, at all host cores and at one thread.  `--impl reference` times the
oracle itself as the reference arm (there is no reference code).
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
    ap.add_argument("--scaling", default="strong", choices=["strong", "weak"],
                    help="strong: the config's global batch split over the ranks; weak: that batch per rank")
    ap.add_argument("--layers", type=int, default=None, help="override layer count (sweeps only)")
    ap.add_argument("--batch", type=int, default=None,
                    help="override the batch (global for --scaling strong, per GPU for weak; sweeps only)")
    ap.add_argument("--prefix", type=int, default=None, help="override prefix (sweeps only)")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--no-early", action="store_true", help="plain attention launches (no EARLY_PREFIX)")
    ap.add_argument("--verify", default=None, help="comma list overriding the config's verify modes")
    ap.add_argument("--gather", default="auto", choices=["auto", "p2p", "nccl"],
                    help="tokens-only exchange: fused into the verifier with peer stores (NEXT-4a) or an NCCL "
                         "all-gather between the verify and commit graphs (the baseline); auto = p2p when there "
                         "is something to exchange (N > 1 or kv-head sharding), else none")
    ap.add_argument("--shard", default="auto", choices=["auto", "request", "kv"],
                    help="layout: request sharding, or kv-head sharding (GQA; auto for G > 1 at N > 1)")
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
# workload: this rank's share of the global problem
# ------------------------------------------------------------------------------------------
def global_batch(cfg: W.Config, args, ws: int) -> int:
    b = args.batch or cfg.batch
    return b * ws if args.scaling == "weak" else b


def use_kv_shard(cfg: W.Config, args, ws: int) -> bool:
    G = cfg.num_q_heads // cfg.num_kv_heads
    if args.shard == "kv":
        return True
    return ws > 1 and args.shard == "auto" and G > 1 and cfg.num_kv_heads % ws == 0


class Workload:
    """One rank's inputs (step.Layout): the attention batch (its requests, or all requests for its
    kv-head shard) and the verification batch (its requests), generated per global request id."""

    def __init__(self, cfg: W.Config, args, layout, device):
        self.cfg, self.layout = cfg, layout
        self.L = args.layers or cfg.layers
        self.P = args.prefix or cfg.prefix
        self.V = cfg.vocab
        self.verify = tuple(args.verify.split(",")) if args.verify else cfg.verify
        parent, depth = cfg.tree
        self.N = int(parent.shape[0])
        self.Dmax = cfg.max_depth
        self.smax = self.P + self.N
        self.Hq, self.Hkv = layout.nq, layout.nkv
        self.tb = W.make_tree_batch([(parent, depth)] * layout.attn_cnt, [self.P] * layout.attn_cnt,
                                    device=device, max_depth=self.Dmax)
        if layout.kv_shard:
            self.tbv = W.make_tree_batch([(parent, depth)] * layout.req_cnt, [self.P] * layout.req_cnt,
                                         device=device, max_depth=self.Dmax)
        else:
            self.tbv = self.tb
        self.ai = W.make_request_attention_inputs(self.tb, list(layout.attn_ids), self.L, cfg.num_q_heads,
                                                  cfg.num_kv_heads, self.smax, cfg.seed,
                                                  q_heads=(layout.q0, layout.nq), kv_heads=(layout.kv0, layout.nkv),
                                                  device=device)
        # greedy trees take the top-k draft tokens, MSS trees i.i.d. draws (R13: only the latter carry
        # MSS's distributional guarantee), so each verifier gets the tree tokens of its own mode
        self.vi = {m: W.make_request_verify_inputs(self.tbv, list(layout.verify_ids), self.V, cfg.seed, m,
                                                   device=device) for m in self.verify}
        if len(self.vi) > 1:
            # the same LLM logits and SSM distributions (only the tree tokens differ): one copy in HBM
            first = self.vi[self.verify[0]]
            for m in self.verify[1:]:
                assert torch.equal(self.vi[m].logits, first.logits)
                self.vi[m] = W.VerifyInputs(first.logits, first.draft_probs, self.vi[m].tree_tokens)
        self.bytes_launch = self.attn_bytes_per_launch()
        self.flops_launch = self.attn_flops_per_launch()

    def tree_tokens_per_step(self) -> int:
        """Tree tokens this rank verifies per step (its requests)."""
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
        tree_pairs = np.array([int((dep[b, :n[b]] + 1).sum()) for b in range(len(n))])
        return int((4 * 128 * (n * pl + tree_pairs) * self.Hq).sum())


def percentiles(xs, qs=(10, 50, 90)):
    return {f"p{q}": round(float(np.percentile(xs, q)), 4) for q in qs}


def run_ours(args, ws, rank, local):
    import paper_conf_asplos_miaoozcwzwzyssc24_b200 as spi
    from paper_conf_asplos_miaoozcwzwzyssc24_b200 import step as S

    device = torch.device("cuda", local)
    torch.cuda.set_device(device)
    affinity_before = bind_to_gpu_numa_node(local)
    bound_cpus = len(os.sched_getaffinity(0)) if affinity_before else 0
    cfg = W.CONFIGS[args.config]
    Bg = global_batch(cfg, args, ws)
    kv_shard = use_kv_shard(cfg, args, ws)
    layout = S.make_layout(Bg, ws, rank, cfg.num_q_heads, cfg.num_kv_heads, kv_shard)
    wl = Workload(cfg, args, layout, device)
    L, N, Dmax, Lp = wl.L, wl.N, wl.Dmax, wl.Dmax + 1
    shape = spi.make_shape(layout.attn_cnt, N, wl.Hq, wl.Hkv, wl.smax, num_layers=L, vocab=wl.V, max_depth=Dmax)
    shape_v = (spi.make_shape(layout.req_cnt, N, 1, 1, wl.smax, num_layers=L, vocab=wl.V, max_depth=Dmax)
               if kv_shard else shape)
    tree = (wl.tb.parent, wl.tb.depth, wl.tb.prefix_len, wl.tb.n_nodes)
    tree_v = (wl.tbv.parent, wl.tbv.depth, wl.tbv.prefix_len, wl.tbv.n_nodes) if kv_shard else tree
    from paper_conf_asplos_miaoozcwzwzyssc24_b200 import dist as D
    p2p, gather_note = None, "NCCL all_gather_into_tensor between the verify and commit graphs" if ws > 1 else \
        "local copy (N = 1)"
    need_gather = ws > 1 or kv_shard or args.gather != "auto"
    if not need_gather:
        gather_note = "none (N = 1, request-sharded: the verifier's own output is the whole table)"
    if args.gather in ("auto", "p2p") and need_gather:
        try:
            p2p = D.P2PGather(Bg, ws, rank, Lp, device, exchange=D.all_gather_object_exchange if ws > 1 else None)
            gather_note = ("fused into the committed verifier: peer stores of every request's row + epoch flags "
                           "(CUDA IPC over NVLink), device-side wait in the verify graph")
        except Exception as exc:   # (setup only: no IPC between the ranks' GPUs) -> the NCCL baseline
            gather_note = f"p2p setup failed ({type(exc).__name__}: {exc}); NCCL all-gather"
    step = S.VerifyStep(S.DeviceOps(), layout, shape, shape_v, tree, tree_v, wl.verify, Lp, device, p2p=p2p)
    inputs = {m: (wl.vi[m].logits, wl.vi[m].tree_tokens, wl.vi[m].draft_probs if m == "mss" else None)
              for m in wl.verify}
    out = torch.empty_like(wl.ai.q)
    prefix0 = wl.tb.prefix_len.clone()
    early = not args.no_early

    def seg_prepare():
        wl.tb.prefix_len.copy_(prefix0)   # every step verifies a fresh tree over the same prefix
        step.prepare()

    def seg_attention():
        for l in range(L):
            step.attention(wl.ai.q[l], wl.ai.k_cache[l], wl.ai.v_cache[l], out[l], layer=l if early else 0)

    def seg_verify():
        step.verify(inputs, seed=cfg.seed, offset=0)
        if p2p is not None:
            step.gather()    # device-side wait for every rank's rows (graph-capturable)

    def gather_between():
        if p2p is None and need_gather:
            step.gather()    # NCCL / local copy: eager, between the verify and commit graphs

    def seg_commit():
        step.commit(wl.ai.k_cache, wl.ai.v_cache)

    # verify and commit in one graph unless an eager (NCCL) gather sits between them: the commit needs
    # only the committed verifier, so it overlaps the other verifier running on the side stream
    eager_gather = p2p is None and need_gather

    def seg_verify_commit():
        step.verify(inputs, seed=cfg.seed, offset=0, join=False)
        if p2p is not None:
            step.gather()
        step.commit(wl.ai.k_cache, wl.ai.v_cache)
        step.join()

    launches_per_step = (spi.specinfer_launches_per_call("tree_prepare") * (2 if kv_shard else 1) +
                         L * spi.specinfer_launches_per_call("tree_attention") +
                         ("greedy" in wl.verify) * spi.specinfer_launches_per_call("verify_greedy") +
                         ("mss" in wl.verify) * spi.specinfer_launches_per_call("verify_mss") +
                         spi.specinfer_launches_per_call("kv_commit") +
                         (spi.specinfer_launches_per_call("gather_wait") if p2p is not None else 0))

    # ---- capture the segments as CUDA graphs (one launch each per step; the gather stays eager) ----
    s = torch.cuda.Stream(device)
    s.wait_stream(torch.cuda.current_stream(device))
    with torch.cuda.stream(s):
        for _ in range(2):  # eager warm-up (lazy init, tensor-map encode, func attributes)
            seg_prepare(); seg_attention(); seg_verify(); gather_between(); seg_commit()
    torch.cuda.synchronize(device)
    graphs = []
    segs = (seg_prepare, seg_attention, seg_verify, seg_commit) if eager_gather else \
        (seg_prepare, seg_attention, seg_verify_commit)
    for fn in segs:
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g, stream=s):
            fn()
        graphs.append(g)
    torch.cuda.synchronize(device)

    with torch.cuda.stream(s):
        for _ in range(args.warmup):
            graphs[0].replay(); graphs[1].replay(); graphs[2].replay()
            if eager_gather:
                gather_between(); graphs[3].replay()
    torch.cuda.synchronize(device)
    K = args.steps
    ev = [[torch.cuda.Event(enable_timing=True) for _ in range(3)] for _ in range(K)]
    e_all = [torch.cuda.Event(enable_timing=True) for _ in range(2)]
    sampler = ClockSampler(local) if rank == 0 else None
    barrier(ws)
    torch.cuda.synchronize(device)
    if sampler:
        sampler.start()
        time.sleep(0.3)
    with torch.cuda.stream(s):
        e_all[0].record(s)
        for k in range(K):
            ev[k][0].record(s)
            graphs[0].replay()
            ev[k][1].record(s)
            graphs[1].replay()
            ev[k][2].record(s)
            graphs[2].replay()
            if eager_gather:
                gather_between()
                graphs[3].replay()
        e_all[1].record(s)
    torch.cuda.synchronize(device)
    barrier(ws)
    clocks = sampler.stop() if sampler else None
    total_ms = max_over_ranks(e_all[0].elapsed_time(e_all[1]), ws, device)
    step_ms = [ev[k][0].elapsed_time(ev[k + 1][0]) for k in range(K - 1)] + \
              [ev[K - 1][0].elapsed_time(e_all[1])]
    attn_ms = sum(ev[k][1].elapsed_time(ev[k][2]) for k in range(K))
    prep_ms = sum(ev[k][0].elapsed_time(ev[k][1]) for k in range(K)) / K
    post_ms = (sum(ev[k][2].elapsed_time(ev[k + 1][0]) for k in range(K - 1)) +
               ev[K - 1][2].elapsed_time(e_all[1])) / K
    attn_ms_max = max_over_ranks(attn_ms, ws, device)
    ms_per_step = total_ms / K
    tokens_step_global = int(wl.tree_tokens_per_step())
    if ws > 1:
        t = torch.tensor([tokens_step_global], dtype=torch.int64, device=device)
        torch.distributed.all_reduce(t)
        tokens_step_global = int(t.item())
    value = tokens_step_global * K / (total_ms / 1e3)
    na_c = step.accepted()[0]
    acc = {m: float(step.res[m][2].float().mean().item()) for m in wl.verify}

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
        ent = tr.get(f"{args.config}:L{L}:B{layout.attn_cnt}:P{wl.P}") or (tr.get(args.config) if ws == 1 else None)
        if ent:
            traffic = ent["dram_bytes_per_launch"]
    except Exception:
        pass
    # a kernel timed inside a long step takes the sustained tensor figure; the burst one is reported beside
    tf_peak, tf_src = 1590.0, "fallback (B200_PROFILING.md)"
    tf_burst = float(peaks.get("bf16_tflops", 1590.0)) if peaks else 1590.0
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
                    "frac_of_burst_tensor": round(tflops / tf_burst, 4), "burst_tensor_peak": tf_burst,
                    "hbm_gbs": round(achieved, 1), "hbm_frac": round(achieved / peak, 4), "hbm_peak": peak,
                    "hbm_peak_source": peak_src}
    else:
        roofline = {"bound": "hbm", "kernel": kname, "achieved": round(achieved, 1), "peak": peak,
                    "unit": "GB/s", "frac": round(achieved / peak, 4), "traffic": traffic,
                    "peak_source": peak_src, "tensor_tflops": round(tflops, 2),
                    "tensor_frac": round(tflops / tf_peak, 4), "tensor_peak": tf_peak,
                    "tensor_frac_of_burst": round(tflops / tf_burst, 4)}
    # BASELINE.json's north star quotes the KV stream against "about 8 TB/s": context only
    roofline["hbm_frac_of_8TBps"] = round(achieved / 8000.0, 4)
    roofline.update({"algorithmic_bytes_per_launch": bytes_launch, "arithmetic_intensity": round(ai_launch, 1),
                     "avg_launch_us": round(attn_launch_s * 1e6, 2),
                     "share_of_step": round(attn_ms_max / total_ms, 4)})
    # the practical ceiling: the library's TMA read probe over the same K and V bytes (one layer)
    probe_ms = []
    with torch.cuda.stream(s):
        for it in range(6):
            p0, p1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            p0.record(s)
            spi.specinfer_hbm_read_probe(wl.ai.k_cache[it % L])
            spi.specinfer_hbm_read_probe(wl.ai.v_cache[it % L])
            p1.record(s)
            probe_ms.append((p0, p1))
    torch.cuda.synchronize(device)
    probe_s = statistics.median(a.elapsed_time(b) for a, b in probe_ms[1:]) / 1e3
    probe_gbs = 2 * wl.ai.k_cache[0].numel() * 2 / probe_s / 1e9
    roofline["tma_read_probe_gbs"] = round(probe_gbs, 1)
    roofline["hbm_frac_of_tma_probe"] = round(achieved / probe_gbs, 4)

    # ---- end to end through the public API with host buffers ----
    e2e = None
    if not args.no_e2e:
        h_q = torch.empty_like(wl.ai.q, device="cpu").pin_memory()
        h_q.copy_(wl.ai.q)
        # the step's inputs once each: the LLM logits (shared by the verifiers), the draft
        # probabilities (MSS), every verifier's tree tokens
        d_list = [wl.vi[wl.verify[0]].logits] + ([wl.vi["mss"].draft_probs] if "mss" in wl.verify else []) + \
            [wl.vi[m].tree_tokens for m in wl.verify]
        h_list = [t.cpu().pin_memory() for t in d_list]
        tree_dev = [wl.tb.parent, wl.tb.depth, wl.tb.n_nodes, prefix0]
        h_tree = [t.cpu().pin_memory() for t in tree_dev]
        res_a, res_n = step.res[step.commit_mode][1], step.res[step.commit_mode][2]
        h_res_a = torch.empty(tuple(res_a.shape), dtype=torch.int32).pin_memory()
        h_res_n = torch.empty(tuple(res_n.shape), dtype=torch.int32).pin_memory()
        h2d = h_q.numel() * 2 + sum(t.numel() * t.element_size() for t in h_list) + sum(t.numel() * 4 for t in h_tree)
        d2h = h_res_a.numel() * 4 + h_res_n.numel() * 4

        # Pipelined steps (a serving loop's double buffering): the inputs live in two device sets; while
        # step k computes on set k % 2, a copy stream (pinned memory, the copy engines) uploads step
        # k + 1's inputs into the other set, and the step's graph joins that copy at its end.  Every
        # step's inputs still cross PCIe inside the timed region: the first step's before the loop,
        # step k + 1's during step k; the last step uploads nothing.  Each step ends with the D2H read
        # of its result.
        copy_s = torch.cuda.Stream(device)
        ev_fork = torch.cuda.Event()
        live_tree = tree_dev   # the tensors the step's TreeState / VerifyStep hold
        sets = []
        for _ in range(2):
            sets.append({"q": torch.empty_like(wl.ai.q), "list": [torch.empty_like(t) for t in d_list],
                         "tree": [torch.empty_like(t) for t in tree_dev]})
        n_modes = len(wl.verify)

        def set_inputs(st_):
            lg = st_["list"][0]
            dp = st_["list"][1] if "mss" in wl.verify else None
            toks = st_["list"][len(st_["list"]) - n_modes:]
            return {m: (lg, toks[i], dp if m == "mss" else None) for i, m in enumerate(wl.verify)}

        def upload(st_):
            for d, h in zip(st_["tree"], h_tree):
                d.copy_(h, non_blocking=True)
            st_["q"].copy_(h_q, non_blocking=True)
            for d, h in zip(st_["list"], h_list):
                d.copy_(h, non_blocking=True)

        def body(st_):
            for d, src in zip(live_tree, st_["tree"]):
                d.copy_(src)
            seg_prepare()   # (prefix_len reset from the uploaded committed lengths, then tree_prepare)
            for l in range(L):
                step.attention(st_["q"][l], wl.ai.k_cache[l], wl.ai.v_cache[l], out[l], layer=l if early else 0)
            step.verify(set_inputs(st_), seed=cfg.seed, offset=0, join=False)
            if p2p is not None:
                step.gather()
            gather_between()
            seg_commit()
            step.join()
            h_res_a.copy_(res_a, non_blocking=True)
            h_res_n.copy_(res_n, non_blocking=True)

        def e2e_step(k, last):
            cur, nxt = sets[k % 2], sets[(k + 1) % 2]
            if not last:
                ev_fork.record(s)
                copy_s.wait_event(ev_fork)
                with torch.cuda.stream(copy_s):
                    upload(nxt)
            body(cur)
            if not last:
                s.wait_stream(copy_s)

        def prologue():
            upload(sets[0])

        with torch.cuda.stream(s):
            prologue()
            e2e_step(0, False)
            e2e_step(1, True)   # eager warm-up of both sets and of the multi-stream step
        torch.cuda.synchronize(device)
        graphs_e2e = None
        if ws == 1:
            graphs_e2e = {}
            for k in range(2):
                for last in (False, True):
                    g = torch.cuda.CUDAGraph()
                    with torch.cuda.graph(g, stream=s):
                        e2e_step(k, last)
                    graphs_e2e[(k, last)] = g
            torch.cuda.synchronize(device)

        def e2e_run(nsteps):
            prologue()
            for k in range(nsteps):
                last = k == nsteps - 1
                if graphs_e2e is not None:
                    graphs_e2e[(k % 2, last)].replay()
                else:
                    e2e_step(k % 2, last)

        with torch.cuda.stream(s):
            e2e_run(max(2, args.warmup))
        torch.cuda.synchronize(device)
        barrier(ws)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        with torch.cuda.stream(s):
            e0.record(s)
            e2e_run(K)
            e1.record(s)
        torch.cuda.synchronize(device)
        barrier(ws)
        e2e_ms = max_over_ranks(e0.elapsed_time(e1), ws, device)
        e2e = {"value": round(tokens_step_global * K / (e2e_ms / 1e3), 1), "unit": UNIT,
               "h2d_bytes_per_step": int(h2d), "d2h_bytes_per_step": int(d2h),
               "ms_per_step": round(e2e_ms / K, 4),
               "inputs": "per step from pinned host memory: tree arrays, q of every layer, the LLM logits"
                         + (", draft probabilities" if "mss" in wl.verify else "")
                         + ", each verifier's tree tokens; result read back: accepted tokens + counts; two device "
                           "input sets: step k+1's H2D on a copy stream during step k (the first step's before the "
                           "loop, inside the timed region)"}

    cpu = None
    if rank == 0 and ws == 1 and not args.no_cpu:
        wl.tb.prefix_len.copy_(prefix0)   # undo the last step's commit: the sample is a fresh iteration
        torch.cuda.synchronize(device)
        if affinity_before:
            os.sched_setaffinity(0, affinity_before)   # the oracle gets every host core again
        cpu = cpu_baseline(wl)

    line = {
        "metric": METRIC, "value": round(value, 1), "unit": UNIT, "n_gpus": ws, "steps": K,
        "warmup": args.warmup, "ms_per_step": round(ms_per_step, 4), "higher_is_better": True,
        "scaling": args.scaling, "vs_baseline": None, "dtype": "bf16", "data": "synthetic",
        "config": {"workload": f"{cfg.name}: {cfg.description}", "layers": L, "global_batch": Bg,
                   "batch_per_gpu": layout.req_cnt, "prefix": wl.P, "tree_nodes": N, "max_depth": Dmax,
                   "num_q_heads": cfg.num_q_heads, "num_kv_heads": cfg.num_kv_heads, "vocab": wl.V,
                   "verify": list(wl.verify),
                   "parallelism": (f"kv-head-sharded attention/commit x{ws} ({layout.nkv} kv-heads per GPU), "
                                   f"request-sharded verification" if kv_shard
                                   else f"request-sharded x{ws}") if ws > 1 else "single GPU",
                   "l2": "no flush: every step streams this GPU's KV cache "
                         f"({2 * L * layout.attn_cnt * wl.Hkv * wl.smax * 256 / 1e9:.1f} GB) >> 126 MB L2",
                   "graph": ("4 CUDA graphs per step (prepare | L x attention | verify | commit)" if eager_gather else
                             "3 CUDA graphs per step (prepare | L x attention | verify + gather + commit)"),
                   "gather": gather_note,
                   "host_binding": (f"pinned buffers allocated under the GPU-local CPU set ({bound_cpus} "
                                    "CPUs, sysfs local_cpulist)" if affinity_before else "unbound"),
                   "attention_launch": "SPECINFER_ATTN_EARLY_PREFIX on layers >= 1" if early else "plain"},
        "step_ms": percentiles(step_ms),
        "roofline": roofline, "cpu_baseline": cpu, "e2e": e2e,
        "gpu_launches": launches_per_step * K, "clocks": clocks,
        "extra": {"tree_tokens_per_step": tokens_step_global,
                  "mean_n_accepted": acc, "committed_verifier": step.commit_mode,
                  "accepted_tokens_per_s_rank0": round(float(na_c.sum().item()) * K / (total_ms / 1e3), 1),
                  "attention_ms_per_step": round(attn_ms_max / K, 4),
                  "prepare_ms_per_step": round(prep_ms, 4),
                  "verify_gather_commit_ms_per_step": round(post_ms, 4)},
    }
    if rank == 0:
        print(json.dumps(line), flush=True)


# ------------------------------------------------------------------------------------------
# CPU baseline: the fp64 oracle as it stands, on a bounded sample of the same workload
# ------------------------------------------------------------------------------------------
def _oracle_sample(wl: Workload, n_req: int, layers=(0,), threads=None):
    """Times the fp64 oracle (as it stands) on `n_req` requests of the workload: tree attention of the
    given layers, then greedy / MSS verification of those requests.  Returns (attention s,
    verification s, threads used)."""
    import oracle
    cores = threads or len(os.sched_getaffinity(0))
    oracle.set_num_threads(cores)
    tb, tbv = wl.tb, wl.tbv
    par, dep = tb.parent[:n_req].cpu(), tb.depth[:n_req].cpu()
    pl, nn_ = tb.prefix_len[:n_req].cpu(), tb.n_nodes[:n_req].cpu()
    ta = 0.0
    for l in layers:
        q = wl.ai.q[l, :n_req].cpu()
        k = wl.ai.k_cache[l, :n_req].cpu()
        v = wl.ai.v_cache[l, :n_req].cpu()
        t0 = time.perf_counter()
        oracle.tree_attention(q, k, v, par, dep, pl, nn_)
        ta += time.perf_counter() - t0
    nv = min(n_req, tbv.parent.shape[0])
    pv, nnv = tbv.parent[:nv].cpu().numpy(), tbv.n_nodes[:nv].cpu().numpy()
    t1 = time.perf_counter()
    for m, vi in wl.vi.items():
        lg, toks = vi.logits[:nv].cpu().numpy(), vi.tree_tokens[:nv].cpu().numpy()
        if m == "greedy":
            oracle.verify_greedy(lg, toks, pv, nnv, path_len=wl.Dmax + 1)
        else:
            oracle.verify_mss(lg, toks, pv, nnv, vi.draft_probs[:nv].cpu().numpy(), seed=1, path_len=wl.Dmax + 1)
    tv = time.perf_counter() - t1
    return ta, tv, cores


def cpu_baseline(wl: Workload, budget_s: float = 12.0):
    """The oracle timed on the host cores on a bounded sample (~10-20 s): every request of the
    step, as many layers as fit the budget (extrapolated linearly to all layers when fewer); and
    at ONE thread on one request x one layer (scaled to the step)."""
    B = wl.tb.parent.shape[0]
    ta1, tv, cores = _oracle_sample(wl, B, layers=(0,))
    n_layers = int(max(1, min(wl.L, budget_s // max(ta1, 1e-3))))
    if n_layers > 1:
        ta, tv, cores = _oracle_sample(wl, B, layers=tuple(range(n_layers)))
    else:
        ta = ta1
    t_step = ta * wl.L / n_layers + tv
    tokens = wl.tree_tokens_per_step()
    extra = "" if n_layers == wl.L else f", x{wl.L / n_layers:.1f} extrapolated to {wl.L} layers"
    # one thread: one request, one layer (+ its verification), scaled by requests and layers
    t1a, t1v, _ = _oracle_sample(wl, 1, layers=(0,), threads=1)
    t_step1 = (t1a * wl.L + t1v) * B
    return {"value": round(tokens / t_step, 3), "unit": UNIT, "cores": cores, "kind": "oracle",
            "sample": f"all {B} requests, tree attention of {n_layers} of {wl.L} layers "
                      f"({ta:.1f} s fp64{extra}) + greedy/MSS verification ({tv:.2f} s)",
            "one_thread": {"value": round(tokens / t_step1, 4), "unit": UNIT, "cores": 1,
                           "sample": f"1 request x 1 layer ({t1a:.2f} s) + its verification ({t1v:.3f} s), "
                                     f"scaled x{wl.L} layers x {B} requests"}}


def run_reference(args, ws, rank, local):
    """Reference arm: the oracle timed on the host cores (there is no reference code; PAPER.md
    only).  Rank 0 alone runs at N>1.  One reference step = the oracle's pass over ONE layer of the
    arm's whole global batch plus its verification (measured; `ms_per_step` is that time), cycling
    through the layers; `value` extrapolates the layer time to all L layers (labelled)."""
    if rank != 0:
        return
    from paper_conf_asplos_miaoozcwzwzyssc24_b200 import step as S
    cfg = W.CONFIGS[args.config]
    Bg = global_batch(cfg, args, ws)
    device = torch.device("cuda", local) if torch.cuda.is_available() else torch.device("cpu")
    layout = S.make_layout(Bg, 1, 0, cfg.num_q_heads, cfg.num_kv_heads, False)
    wl = Workload(cfg, args, layout, device)
    for _ in range(args.warmup):
        _oracle_sample(wl, Bg, layers=(0,))
    ta_s, tv_s, cores = [], [], 1
    w0 = time.perf_counter()
    for it in range(args.steps):
        ta, tv, cores = _oracle_sample(wl, Bg, layers=(it % wl.L,))
        ta_s.append(ta)
        tv_s.append(tv)
    wall = time.perf_counter() - w0
    tokens = wl.tree_tokens_per_step()
    t_full = statistics.mean(ta_s) * wl.L + statistics.mean(tv_s)
    value = tokens / t_full
    sample = (f"per step: fp64 oracle tree attention of one layer of all {Bg} requests ({statistics.mean(ta_s):.3f} s) "
              f"+ their verification ({statistics.mean(tv_s):.3f} s); value extrapolates the layer to {wl.L} layers")
    print(json.dumps({
        "impl": "reference", "metric": METRIC, "value": round(value, 3), "unit": UNIT, "n_gpus": ws,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(1e3 * wall / args.steps, 3),
        "higher_is_better": True, "scaling": args.scaling, "vs_baseline": None, "dtype": "f64", "data": "synthetic",
        "config": {"workload": f"{cfg.name}: {cfg.description}", "layers": wl.L, "global_batch": Bg,
                   "prefix": wl.P, "tree_nodes": wl.N, "verify": list(wl.verify)},
        "extrapolated": {"seconds_per_full_iteration": round(t_full, 3), "layers_measured_per_step": 1,
                         "layers": wl.L},
        "cpu_baseline": {"value": round(value, 3), "unit": UNIT, "cores": cores, "kind": "oracle", "sample": sample},
        "e2e": {"value": round(value, 3), "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }), flush=True)


def bind_to_gpu_numa_node(local: int):
    """Restrict this process to the CPUs of the GPU's NUMA node (from sysfs) before any pinned host
    buffer is allocated, so first-touch puts them on the node the GPU's PCIe link hangs off (a far node
    cost ~20% of the H2D bandwidth on some boxes).  Returns the previous affinity set (restored for
    the CPU baseline), or None when the topology is not available."""
    try:
        pr = torch.cuda.get_device_properties(local)
        bdf = f"{pr.pci_domain_id:04x}:{pr.pci_bus_id:02x}:{pr.pci_device_id:02x}.0"
        with open(f"/sys/bus/pci/devices/{bdf}/local_cpulist") as f:
            spec = f.read().strip()
        cpus = set()
        for part in spec.split(","):
            lo, _, hi = part.partition("-")
            cpus.update(range(int(lo), int(hi or lo) + 1))
        before = os.sched_getaffinity(0)
        cpus &= before
        if cpus and cpus != before:
            os.sched_setaffinity(0, cpus)
            return before
    except Exception:
        pass
    return None


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
