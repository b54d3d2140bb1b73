timeout 900 python -m pytest tests/test_gpu_seqdec.py tests/test_gpu_ns.py -x -q > gpurun_out/pyt_next.log 2>&1; echo pytest=$?; tail -5 gpurun_out/pyt_next.log
timeout 600 python tools/mss_vs_ns.py --out gpurun_out/mss_vs_ns.jsonl
timeout 900 python tools/fig11_ablation.py --out gpurun_out/fig11.jsonl
