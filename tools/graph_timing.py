"""Per-launch device time of a chain of launches replayed from one CUDA graph (development tools):
the launches rotate over enough distinct input buffers that the bytes they stream exceed the 126 MB
L2 (no flush kernel in the timed region), exactly as consecutive layers run inside bench.py."""
import torch


def layers_for(bytes_per_layer: int, target: int = 512 << 20, cap: int = 64) -> int:
    """Number of distinct buffers (layers) whose total exceeds `target` bytes (>= 4x the L2)."""
    return int(max(1, min(cap, -(-target // max(bytes_per_layer, 1)))))


def graph_us_per_launch(launch, n_buffers: int, reps: int = None, warm: int = 2) -> float:
    """launch(i, first) issues launch number i (buffer i % n_buffers; `first` marks the chain's first
    launch, e.g. to skip SPECINFER_ATTN_EARLY_PREFIX); returns the median over 3 timed replays of
    (graph time / launches)."""
    reps = reps or max(n_buffers, 16)
    s = torch.cuda.Stream()
    s.wait_stream(torch.cuda.current_stream())
    with torch.cuda.stream(s):
        for i in range(min(reps, 4)):
            launch(i, i == 0)
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=s):
        for i in range(reps):
            launch(i, i == 0)
    for _ in range(warm):
        g.replay()
    torch.cuda.synchronize()
    ts = []
    for _ in range(3):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        with torch.cuda.stream(s):
            e0.record(s)
            g.replay()
            e1.record(s)
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1) * 1e3 / reps)
    ts.sort()
    return ts[1]
