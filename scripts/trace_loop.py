"""Phase timeline of the persistent TED loop kernel (BTED_FLAG_PERSISTENT_LOOP,
eager launch, BTED_TRACE): per step, the spread over CTAs of each phase.
Usage (GPU box): python scripts/trace_loop.py [N] [out.txt]"""
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
N = int(sys.argv[1]) if len(sys.argv) > 1 else 16384
path = "/tmp/bted_trace.bin"
if os.path.exists(path):
    os.unlink(path)
os.environ["BTED_TRACE"] = path
import paper_conf_date_sunbg021_b200 as bt  # noqa: E402
from paper_conf_date_sunbg021_b200 import _lib as L  # noqa: E402
from synth import uniform_pool, median_gamma  # noqa: E402

X = uniform_pool(N, 16, 1)
g = median_gamma(X, 1)
flags = L.BTED_FLAG_PERSISTENT_LOOP | L.BTED_FLAG_NO_GRAPH | L.BTED_FLAG_NO_SMALL
with bt.CandidateSet(X, g, flags=flags) as cs:
    for _ in range(3):
        cs.select(64, 0.1)
raw = open(path, "rb").read()
hdr = np.frombuffer(raw[:12], np.int32)
grid, m, k = (int(x) for x in hdr)
rec = 12 + grid * m * k * 8
arr = np.frombuffer(raw[len(raw) - rec + 12:], np.uint64).reshape(grid, m, k).astype(np.int64)
names = ["E wait fin_done", "E ell units", "H (ell_done + h cols)", "T tiles", "F wait tdone+h", "F fin units"]
out = [f"N={N} grid={grid} m={m}; per step, over CTAs: median / max [us] of each phase"]
steps = range(2, m - 1)
tot = np.zeros(len(names))
for t in steps:
    d = np.diff(arr[:, t, :7], axis=1) / 1e3                 # [grid][6]
    tot += np.median(d, axis=0)
for i, nm in enumerate(names):
    allv = np.concatenate([np.diff(arr[:, t, :7], axis=1)[:, i] / 1e3 for t in steps])
    out.append(f"{nm:28s} median {np.median(allv):8.2f}  p90 {np.percentile(allv, 90):8.2f}  max {allv.max():8.2f}")
step_ns = [(arr[:, t + 1, 0].min() - arr[:, t, 0].min()) / 1e3 for t in steps]
out.append(f"step (E start to E start, earliest CTA): median {np.median(step_ns):.2f} us")
tile_end_spread = [(arr[:, t, 4].max() - arr[:, t, 4].min()) / 1e3 for t in steps]
out.append(f"T end spread over CTAs: median {np.median(tile_end_spread):.2f} us")
txt = "\n".join(out)
print(txt)
if len(sys.argv) > 2:
    open(sys.argv[2], "w").write(txt + "\n")
