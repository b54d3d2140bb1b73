#!/bin/bash
# A/B of the swapped kernel's split merge: GPU tests, per-launch C2 at B = 1, 4, 16 for each lib, tail of one launch.
mkdir -p gpurun_out
timeout 900 python -m pytest tests -x -q -m gpu > gpurun_out/pytest_gpu.log 2>&1; echo pytest=$?; tail -2 gpurun_out/pytest_gpu.log
for lib in abtest/lib_*.so; do
  echo "== $lib"
  for b in 1 4 16; do timeout 120 python tools/attn_probe.py --config C2 --batch $b --layers 4 --iters 40 --lib $lib; done
  timeout 120 python tools/attn_probe.py --config C1 --layers 1 --iters 40 --lib $lib
done


