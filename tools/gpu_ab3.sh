#!/bin/bash
# A/B of libspecinfer builds in abtest/ on the rows kernel (C3, C4) + GPU parity tests of the tree.
mkdir -p gpurun_out
timeout 900 python -m pytest tests -x -q -m gpu > gpurun_out/pytest_gpu.log 2>&1; echo pytest=$?; tail -3 gpurun_out/pytest_gpu.log
for lib in abtest/lib_*.so; do
  echo "== $lib"
  for c in C3 C4; do timeout 120 python tools/attn_probe.py --config $c --layers 2 --iters 10 --lib $lib; done
  timeout 120 python tools/attn_sweep.py --ns 128,256 --batch 8 --prefix 2048 --iters 10 --lib $lib 2>/dev/null || true
done
timeout 300 python tools/attn_probe.py --config C3 --layers 2 --iters 6 --trace --raw > gpurun_out/trace_C3_new.log 2>&1
