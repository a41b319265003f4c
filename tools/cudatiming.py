"""Device-time measurement of one reduction call, shared by tools/tune.py and bench.py.

`time_calls(launch, regions, ...)` captures R calls (one per input region) into a
CUDA graph and times one replay with CUDA events on the capture stream: host
launch overhead is excluded, kernel-to-kernel gaps inside the graph are not.
Two disjoint region sets are used — one for the warm-up replay (instruction
cache, lazy module load) and one for the timed replay — so every timed call
reads bytes nobody touched recently: with R·S bytes per set > L2 the data
comes from HBM ("cold"); `warm=True` instead re-reads one region (L2-resident
when it fits).
"""
from __future__ import annotations


def time_calls(launch, regions_warm, regions_timed, stream, repeats: int = 1):
    """launch(region) enqueues one call on `stream`.  Returns seconds per call."""
    import torch
    graphs = []
    for regs in (regions_warm, regions_timed):
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g, stream=stream):
            for r in regs:
                launch(r)
        graphs.append(g)
    best = None
    for _ in range(repeats):
        with torch.cuda.stream(stream):  # replay() launches on the current stream
            graphs[0].replay()
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record(stream)
            graphs[1].replay()
            b.record(stream)
        b.synchronize()
        t = a.elapsed_time(b) * 1e-3 / len(regions_timed)
        best = t if best is None else min(best, t)
    return best


def disjoint_regions(pool, count: int, elems: int, align_elems: int = 64):
    """Split `pool` (1-D tensor) into up to 2*count disjoint slices of `elems`
    elements (starts rounded to align_elems); returns (warm_set, timed_set)."""
    stride = (elems + align_elems - 1) // align_elems * align_elems
    fit = pool.numel() // max(stride, 1)
    if fit < 2:  # one region only: the caller uses this for arrays larger than L2
        r = pool[:elems]
        return [r] * count, [r] * count
    per = max(1, min(count, fit // 2))
    regs = [pool[i * stride:i * stride + elems] for i in range(2 * per)]
    warm, timed = regs[:per], regs[per:2 * per]
    # too few disjoint regions: cycle through them (only done when the caller
    # asks for more calls than fit, i.e. for regions far larger than L2)
    return [warm[i % per] for i in range(count)], [timed[i % per] for i in range(count)]
