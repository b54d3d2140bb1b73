#!/bin/bash
# C5 sweep + rows-kernel evidence (ncu --set full at C3 and C4, pipeline trace). Outputs in gpurun_out/.
mkdir -p gpurun_out
timeout 900 python tools/c5_sweep.py --out gpurun_out/c5_sweep.jsonl > gpurun_out/c5_sweep.log 2>&1; echo c5=$?; tail -2 gpurun_out/c5_sweep.log
for c in C3 C4; do
  timeout 600 python tools/attn_probe.py --config $c --layers 2 --iters 6 --trace --raw > gpurun_out/trace_$c.log 2>&1; echo trace$c=$?
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:tree_attn -s 2 -c 1 \
    -o gpurun_out/rows_full_$c python tools/attn_probe.py --config $c --layers 2 --iters 2 > gpurun_out/rows_full_$c.log 2>&1; echo ncu$c=$?
  ncu -i gpurun_out/rows_full_$c.ncu-rep --page raw --csv > gpurun_out/rows_full_${c}_raw.csv 2>/dev/null
  ncu -i gpurun_out/rows_full_$c.ncu-rep --page details --csv > gpurun_out/rows_full_${c}_details.csv 2>/dev/null
  ncu -i gpurun_out/rows_full_$c.ncu-rep --page source --csv > gpurun_out/rows_full_${c}_source.csv 2>/dev/null
done
