#!/bin/bash
# Profiling pass for one round (run under gpurun; single GPU).  Outputs go to gpurun_out/.
#   1. launch list of the bench step (every kernel with its device time; cold-cache, serialised)
#   2. one `ncu --set full` capture of the swapped tree-attention kernel at C2 and of the rows kernel at C3 and C4
#   3. the verify / commit / prepare kernels at C2 (details pages)
set -u
R=${1:-r02}
mkdir -p gpurun_out
timeout -s KILL 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
  --log-file gpurun_out/launches_${R}.csv python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu \
  > gpurun_out/launches_${R}.log 2>&1
timeout -s KILL 900 ncu --set full --clock-control none --import-source on -k regex:tree_attn_kernel -s 3 -c 1 \
  -o gpurun_out/attn_full_${R} python tools/attn_probe.py --layers 4 --iters 4 > gpurun_out/attn_full_${R}.log 2>&1
ncu -i gpurun_out/attn_full_${R}.ncu-rep --page raw --csv > gpurun_out/attn_full_${R}_raw.csv 2>/dev/null
timeout -s KILL 900 ncu --set full --clock-control none --import-source on -k regex:tree_attn_rows -s 2 -c 1 \
  -o gpurun_out/rows_full_C3_${R} python tools/attn_probe.py --config C3 --layers 2 --iters 4 > gpurun_out/rows_full_C3_${R}.log 2>&1
ncu -i gpurun_out/rows_full_C3_${R}.ncu-rep --page raw --csv > gpurun_out/rows_full_C3_${R}_raw.csv 2>/dev/null
timeout -s KILL 900 ncu --set full --clock-control none --import-source on -k regex:tree_attn_rows -s 2 -c 1 \
  -o gpurun_out/rows_full_C4_${R} python tools/attn_probe.py --config C4 --layers 2 --iters 4 > gpurun_out/rows_full_C4_${R}.log 2>&1
ncu -i gpurun_out/rows_full_C4_${R}.ncu-rep --page raw --csv > gpurun_out/rows_full_C4_${R}_raw.csv 2>/dev/null
for k in verify_mss verify_greedy kv_commit tree_validate gather_wait; do
  timeout -s KILL 300 ncu --set full --clock-control none -k regex:$k -c 1 -o gpurun_out/${k}_${R} \
    python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu --layers 1 > /dev/null 2>&1
  ncu -i gpurun_out/${k}_${R}.ncu-rep --page details --csv > gpurun_out/${k}_${R}_details.csv 2>/dev/null
done
echo done
