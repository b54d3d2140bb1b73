"""Summarise the ncu outputs of tools/profile_round.sh (gpurun_out/) into profiles/ (tracked).

    python tools/summarize_profiles.py r01
Writes profiles/<round>_launches.csv (our kernels only: launch order, name, device time),
profiles/<round>_ncu_summary.md and updates profiles/ncu_traffic.json (DRAM bytes per launch of the
tree-attention kernel, read by bench.py for the `roofline.traffic` field).
"""
import collections
import csv
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
R = sys.argv[1] if len(sys.argv) > 1 else "r01"
OUT = os.path.join(ROOT, "gpurun_out")
PROF = os.path.join(ROOT, "profiles")
os.makedirs(PROF, exist_ok=True)


def read_launches(path):
    rows = list(csv.reader(open(path)))
    hi = [i for i, r in enumerate(rows) if r and r[0] == "ID"][0]
    hdr, data = rows[hi], rows[hi + 1:]
    ki, vi = hdr.index("Kernel Name"), hdr.index("Metric Value")
    out = []
    for r in data:
        if "specinfer" in r[ki]:
            out.append((r[0], r[ki].split("(")[0].replace("void ", ""), float(r[vi].replace(",", "")) / 1e3))
    return out


def read_raw(path):
    rows = list(csv.reader(open(path)))
    return {h: (v, u) for h, u, v in zip(rows[0], rows[1], rows[2])}


lines = [f"# ncu summary, round {R[1:]}", ""]
launch_csv = os.path.join(OUT, f"launches_{R}.csv")
if os.path.exists(launch_csv):
    launches = read_launches(launch_csv)
    with open(os.path.join(PROF, f"{R}_launches.csv"), "w", newline="") as f:
        w = csv.writer(f)
        w.writerow(["ncu_id", "kernel", "gpu_time_us"])
        w.writerows([(i, k, f"{t:.3f}") for i, k, t in launches])
    agg = collections.defaultdict(list)
    for _, k, t in launches:
        agg[k].append(t)
    # the HBM read probe (bench.py's practical-ceiling measurement) runs outside the timed step
    outside = {k for k in agg if "hbm_read_probe" in k}
    total = sum(t for _, k, t in launches if k not in outside)
    lines += ["## Launch list (`ncu --metrics gpu__time_duration.sum --clock-control none`, "
              "`bench.py --steps 2 --warmup 1`; cold-cache, serialised)", "",
              "| kernel | launches | mean µs | share of the step's kernel time |", "|---|---|---|---|"]
    for k, v in sorted(agg.items(), key=lambda kv: -sum(kv[1])):
        share = "outside the step (roofline probe)" if k in outside else f"{sum(v) / total:.1%}"
        lines.append(f"| `{k}` | {len(v)} | {sum(v) / len(v):.2f} | {share} |")
    lines.append("")

raw_csv = os.path.join(OUT, f"attn_full_{R}_raw.csv")
traffic = {}
if os.path.exists(raw_csv):
    raw = read_raw(raw_csv)
    keys = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
            "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "lts__t_sector_hit_rate.pct",
            "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active",
            "sm__inst_executed_pipe_xu.avg.pct_of_peak_sustained_active", "launch__registers_per_thread",
            "launch__grid_size", "launch__block_size", "sm__warps_active.avg.pct_of_peak_sustained_active"]
    lines += ["## tree_attn_kernel, `ncu --set full` (C2 shape, one launch = one layer)", "",
              "| metric | value |", "|---|---|"]
    for k in keys:
        if k in raw:
            lines.append(f"| `{k}` | {raw[k][0]} {raw[k][1]} |")
    def to_bytes(v, u):
        scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}[u]
        return float(v.replace(",", "")) * scale
    rd = to_bytes(*raw["dram__bytes_read.sum"])
    wr = to_bytes(*raw["dram__bytes_write.sum"])
    alg = 547880960
    lines += ["", f"DRAM traffic per launch {rd + wr:,.0f} B vs algorithmic {alg:,} B "
              f"(ratio {(rd + wr) / alg:.3f}): every KV byte is read once.", ""]
    traffic = {"C2": {"dram_bytes_per_launch": int(rd + wr), "round": R,
                      "source": f"gpurun_out/attn_full_{R}.ncu-rep (ncu --set full)"}}
    path = os.path.join(PROF, "ncu_traffic.json")
    old = json.load(open(path)) if os.path.exists(path) else {}
    old.update(traffic)
    json.dump(old, open(path, "w"), indent=1)

for cfg_name, alg in (("C3", 612368384), ("C4", 2734161920)):
  # C3: K and V of 32 x 8 (request, kv-head) streams of 4096 + 64 rows, q in, out;
  # C4: 64 x 56 streams of 1024 + 233 rows, q in, out (bench.py's algorithmic_bytes_per_launch)
  rows_csv = os.path.join(OUT, f"rows_full_{cfg_name}_{R}_raw.csv")
  if os.path.exists(rows_csv):
      raw = read_raw(rows_csv)
      keys = ["gpu__time_duration.sum", "sm__cycles_elapsed.avg.per_second", "dram__bytes_read.sum",
              "dram__bytes_write.sum", "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active",
              "sm__inst_executed_pipe_xu.avg.pct_of_peak_sustained_active",
              "sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active",
              "smsp__issue_active.avg.pct_of_peak_sustained_active", "launch__registers_per_thread",
              "launch__grid_size", "launch__block_size"]
      lines += [f"## tree_attn_rows_kernel, `ncu --set full` ({cfg_name} shape, one launch = one layer)", "",
                "| metric | value |", "|---|---|"]
      for k in keys:
          if k in raw:
              lines.append(f"| `{k}` | {raw[k][0]} {raw[k][1]} |")
      def to_bytes(v, u):
          return float(v.replace(",", "")) * {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}[u]
      rd, wr = to_bytes(*raw["dram__bytes_read.sum"]), to_bytes(*raw["dram__bytes_write.sum"])
      lines += ["", f"DRAM traffic per launch {rd + wr:,.0f} B vs algorithmic {alg:,} B (ratio {(rd + wr) / alg:.3f}).", ""]
      path = os.path.join(PROF, "ncu_traffic.json")
      old = json.load(open(path)) if os.path.exists(path) else {}
      old[cfg_name] = {"dram_bytes_per_launch": int(rd + wr), "round": R,
                   "source": f"gpurun_out/rows_full_{cfg_name}_{R}.ncu-rep (ncu --set full)"}
      json.dump(old, open(path, "w"), indent=1)

det_lines = []
for k in ("verify_mss", "verify_greedy", "kv_commit", "tree_validate", "gather_wait"):
    p = os.path.join(OUT, f"{k}_{R}_details.csv")
    if not os.path.exists(p):
        continue
    rows = list(csv.reader(open(p)))
    if not rows or "Metric Name" not in rows[0]:
        continue   # (no launch of that kernel in the profiled run)
    h = rows[0]
    mi, vi, ui = h.index("Metric Name"), h.index("Metric Value"), h.index("Metric Unit")
    vals = {r[mi]: (r[vi], r[ui]) for r in rows[1:]}
    sel = ["Duration", "DRAM Throughput", "Memory Throughput", "Achieved Occupancy", "Registers Per Thread"]
    det_lines.append(f"| `{k}` | " + " | ".join(f"{vals.get(s, ('-', ''))[0]} {vals.get(s, ('', ''))[1]}" for s in sel) + " |")
if det_lines:
    lines += ["## Other kernels (`ncu --set full`, one launch each)", "",
              "| kernel | duration | DRAM throughput | memory throughput | achieved occupancy | registers |",
              "|---|---|---|---|---|---|"] + det_lines + [""]
open(os.path.join(PROF, f"{R}_ncu_summary.md"), "w").write("\n".join(lines))
print("\n".join(lines))
