# quick attention check: parity tests of the attention kernels + per-launch probe timings + ncu counters
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "attention or config" > gpurun_out/pyt2.log 2>&1; echo pytest=$?; tail -3 gpurun_out/pyt2.log
for c in C3 C4 C2; do timeout 120 python tools/attn_probe.py --config $c --layers 4 --iters 20; done
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct,sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active,sm__inst_executed_pipe_xu.avg.pct_of_peak_sustained_active
for c in C3 C4; do timeout 300 ncu --metrics $M --clock-control none -k regex:tree_attn -s 2 -c 1 python tools/attn_probe.py --config $c --layers 2 --iters 2 2>&1 | grep -E "dram__|gpu__time|lts__|tensor|xu"; done
