timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu > gpurun_out/b_c2.json 2> gpurun_out/b_c2.err; tail -2 gpurun_out/b_c2.err
timeout 300 python bench.py --config C3 --steps 3 --warmup 3 --no-cpu --no-e2e --layers 8 > gpurun_out/b_c3r.json 2> gpurun_out/b_c3r.err; tail -2 gpurun_out/b_c3r.err
timeout 300 python bench.py --config C3 --steps 3 --warmup 3 --no-cpu --shard kv --layers 8 > gpurun_out/b_c3k.json 2> gpurun_out/b_c3k.err; tail -2 gpurun_out/b_c3k.err
python - <<'PY'
import json
for f in ["b_c2","b_c3r","b_c3k"]:
    try:
        d=json.load(open(f"gpurun_out/{f}.json"))
        print(f, d["value"], d["ms_per_step"], d["roofline"]["frac"], d["config"]["parallelism"], d["extra"], (d.get("e2e") or {}).get("value"))
    except Exception as e: print(f, "ERR", e)
PY
