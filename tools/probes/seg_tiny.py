"""Segmented (offsets) throughput for very short segments: every group vs the
element-balanced default (graph-timed, 256 MB of fp32 per call)."""
import json
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tools"))
import paper_conf_cgo_gonzalohghmh19_b200 as rb  # noqa: E402
from cudatiming import time_calls  # noqa: E402

dev = torch.device("cuda", 0)
stream = torch.cuda.Stream(dev)
rb.prepare(stream, 1 << 20)
total = (256 << 20) // 4
x = torch.rand(total, device=dev)
rng = np.random.Generator(np.random.PCG64(1))
for name, lens_fn in (("ones", lambda k: np.ones(k, np.int64)), ("0..4", lambda k: rng.integers(0, 5, k)),
                      ("0..16", lambda k: rng.integers(0, 17, k)), ("0..32", lambda k: rng.integers(0, 33, k))):
    mean = {"ones": 1, "0..4": 2, "0..16": 8, "0..32": 16}[name]
    nseg = min(total // mean, (1 << 26))
    lens = lens_fn(nseg)
    offs = np.minimum(np.concatenate([[0], np.cumsum(lens)]), total)
    ot = torch.from_numpy(offs).to(dev)
    xs = x[: int(offs[-1])]
    ob = torch.empty(nseg, device=dev)
    for g in (0, 1, 3, 4):
        def launch(t, g=g):
            rb.reduce_segmented(xs, ot, "sum", out=ob, stream=stream, seg_group=g)
        sec = time_calls(launch, [xs] * 2, [xs] * 5, stream, repeats=2)
        print(json.dumps({"lengths": name, "nseg": nseg, "group": {0: "auto", 1: "warp", 3: "8-lane", 4: "thread"}[g],
                          "us": round(sec * 1e6, 1), "GBps": round(int(offs[-1]) * 4 / sec / 1e9, 1),
                          "segments_per_us": round(nseg / sec / 1e6, 1)}), flush=True)
