"""Where does the end-to-end (host-timed, pool H2D every step) resnet18 number lose against the
device-timed one?  Times K BTED calls five ways: device events on one ctx (bench.py's value),
host clock on one ctx, host clock alternating two ctxs, + the pool H2D (bted_update) of the next
step on the other ctx (bench.py's e2e), + H2D without the device finiteness check."""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_date_sunbg021_b200 as bt  # noqa: E402
from paper_conf_date_sunbg021_b200 import _lib as L  # noqa: E402
from synth import config_pool  # noqa: E402

X, gamma, cfg = config_pool("resnet18")
mu = float(np.float32(cfg["mu"]))
M, m, B = cfg["M"], cfg["m"], cfg["B"]
K = 12
dev = torch.device("cuda", 0)
pins = []
ctxs = []
strs = []
for q in range(2):
    pa = L.PinnedArray(X.shape)
    pa.array[:] = X
    s = torch.cuda.Stream(dev)
    pins.append(pa)
    strs.append(s)
    ctxs.append(bt.CandidateSet(pa.array, gamma, num_batches=B, seed=cfg["seed"], device=0, stream=s.cuda_stream))
for c in ctxs:
    for _ in range(3):
        c.run_batches(M, m, mu, want_batches=False)
res = {}
# device events, one ctx
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
torch.cuda.synchronize()
e0.record(strs[0])
for k in range(K):
    ctxs[0].run_batches(M, m, mu, want_batches=False)
e1.record(strs[0])
torch.cuda.synchronize()
res["device_events_one_ctx_ms"] = e0.elapsed_time(e1) / K


def host(fn):
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    for k in range(K):
        fn(k)
    torch.cuda.synchronize()
    return (time.perf_counter() - t0) * 1e3 / K


res["host_one_ctx_ms"] = host(lambda k: ctxs[0].run_batches(M, m, mu, want_batches=False))
res["host_two_ctx_ms"] = host(lambda k: ctxs[k % 2].run_batches(M, m, mu, want_batches=False))


def with_update(k):
    L.bted_update(ctxs[(k + 1) % 2].ctx, pins[(k + 1) % 2].ptr)
    ctxs[k % 2].run_batches(M, m, mu, want_batches=False)


res["host_two_ctx_h2d_ms"] = host(with_update)
# the same calls, each bracketed by events AND the host clock
evs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(K)]
hts = []
torch.cuda.synchronize()
for k in range(K):
    t0 = time.perf_counter()
    evs[k][0].record(strs[0])
    ctxs[0].run_batches(M, m, mu, want_batches=False)
    evs[k][1].record(strs[0])
    hts.append((time.perf_counter() - t0) * 1e3)
torch.cuda.synchronize()
res["per_call_event_ms"] = float(np.mean([a.elapsed_time(b) for a, b in evs]))
res["per_call_host_ms"] = float(np.mean(hts))
res["event_span_per_call_ms"] = evs[0][0].elapsed_time(evs[-1][1]) / K
print(json.dumps(res))
