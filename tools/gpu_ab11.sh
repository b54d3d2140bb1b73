#!/bin/bash
timeout 600 python -m pytest tests -x -q -m gpu > gpurun_out/pytest_gpu.log 2>&1; echo pytest=$?; tail -1 gpurun_out/pytest_gpu.log
for lib in abtest/lib_*.so; do
  echo "== $lib"
  for b in 4 8 12 16; do timeout 120 python tools/attn_probe.py --config C2 --batch $b --layers 4 --iters 40 --lib $lib; done
  timeout 120 python tools/attn_probe.py --config C4 --layers 2 --iters 10 --lib $lib
  timeout 120 python tools/attn_probe.py --config C3 --layers 2 --iters 10 --lib $lib
done
