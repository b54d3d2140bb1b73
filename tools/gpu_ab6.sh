#!/bin/bash
timeout 600 python -m pytest tests -x -q -m gpu > gpurun_out/pytest_gpu.log 2>&1; echo pytest=$?; tail -1 gpurun_out/pytest_gpu.log
bash tools/gpu_ab5.sh
timeout 120 python tools/attn_sweep.py --ns 128,256 --batch 8 --prefix 2048 --iters 10 --lib abtest/lib_stw.so
timeout 120 python tools/attn_sweep.py --ns 128,256 --batch 8 --prefix 2048 --iters 10 --lib abtest/lib_base.so
