timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "attention or config" > gpurun_out/pyt_ab.log 2>&1; echo pytest=$?; tail -1 gpurun_out/pyt_ab.log
for lib in abtest/lib_*.so; do
  echo "== $lib"; timeout 120 python tools/attn_probe.py --config C2 --expansion 1,1,5,1,1,1,1,1 --layers 4 --iters 20 --lib $lib
  timeout 120 python tools/attn_probe.py --config C2 --layers 4 --iters 20 --lib $lib
done
