# A/B of libspecinfer builds under abtest/ on the attention probe (same box, interleaved)
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "attention or config" > gpurun_out/pyt_ab.log 2>&1; echo pytest=$?; tail -1 gpurun_out/pyt_ab.log
for rep in 1 2; do
for c in C3 C4; do
for lib in abtest/lib_*.so; do
  echo -n "$lib "; timeout 120 python tools/attn_probe.py --config $c --layers 4 --iters 20 --lib $lib
done; done; done
