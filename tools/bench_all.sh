# Bench lines for the round summary (one B200): C2 (the metric's config), C1, C3, C4 and the C2 batch sweep.
# Run under gpurun from the repo root; lines land in gpurun_out/b_*.log.
mkdir -p gpurun_out
python bench.py > gpurun_out/b_c2.log 2>&1
python bench.py --config C1 > gpurun_out/b_c1.log 2>&1
python bench.py --config C3 --steps 10 --warmup 3 > gpurun_out/b_c3.log 2>&1
python bench.py --config C4 --steps 10 --warmup 3 > gpurun_out/b_c4.log 2>&1
for b in 1 2 4 8; do python bench.py --batch $b > gpurun_out/b_c2_b$b.log 2>&1; done
for f in c2 c1 c3 c4 c2_b1 c2_b2 c2_b4 c2_b8; do tail -n 1 gpurun_out/b_$f.log | cut -c1-200; done
