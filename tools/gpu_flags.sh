for f in 0 1 2 4 8 12 3; do timeout 120 python tools/attn_probe.py --config C3 --layers 2 --iters 10 --flags $f; done
