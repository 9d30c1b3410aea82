"""How much of one resnet18 BTED call (bench.py's step) is GPU idle time spent waiting
for the host to enqueue?  Times the call with CUDA events (a) as bench.py runs it and
(b) behind a ~5 ms busy kernel on the same stream, so the host has enqueued the whole
call before the GPU reaches it.  The difference is the host-side gap."""
import json
import os
import sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import paper_conf_date_sunbg021_b200 as bt
from paper_conf_date_sunbg021_b200 import _lib as L
from synth import config_pool

X, gamma, cfg = config_pool("resnet18")
mu = float(np.float32(cfg["mu"]))
dev = torch.device("cuda", 0)
stream = torch.cuda.Stream(dev)
X_dev = torch.from_numpy(X).to(dev)
pool = bt.CandidateSet(X_dev, gamma, num_batches=cfg["B"], seed=cfg["seed"], device=0,
                       flags=L.BTED_FLAG_TIMING, stream=stream.cuda_stream)
M, m = cfg["M"], cfg["m"]
for _ in range(3):
    pool.run_batches(M, m, mu, want_batches=False)
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
res = {"plain": [], "behind_busy_kernel": []}
for it in range(10):
    for mode in res:
        torch.cuda.synchronize()
        if mode == "behind_busy_kernel":
            with torch.cuda.stream(stream):
                torch.cuda._sleep(12_000_000)
        e0.record(stream)
        pool.run_batches(M, m, mu, want_batches=False)
        e1.record(stream)
        torch.cuda.synchronize()
        res[mode].append(e0.elapsed_time(e1))
out = {k: {"median_ms": float(np.median(v)), "min_ms": float(np.min(v))} for k, v in res.items()}
out["gap_ms"] = out["plain"]["median_ms"] - out["behind_busy_kernel"]["median_ms"]
print(json.dumps(out))
