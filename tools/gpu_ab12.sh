#!/bin/bash
timeout 600 python -m pytest tests -x -q -m gpu > gpurun_out/pytest_gpu.log 2>&1; echo pytest=$?; tail -1 gpurun_out/pytest_gpu.log
for rep in 1 2; do for lib in abtest/lib_*.so; do
  echo "== $lib"
  for c in C3 C4; do timeout 120 python tools/attn_probe.py --config $c --layers 2 --iters 10 --lib $lib; done
  timeout 120 python tools/attn_sweep.py --ns 128,256 --batch 8 --prefix 8192 --iters 10 --lib $lib
done; done
