"""Repeat the same selects many times (default streaming engine and the opt-in recomputing
pass) and report any run whose picks or fp32 score bits differ from the first: a race in a
PDL-chained step would show up as run-to-run differences."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402

import paper_conf_date_sunbg021_b200 as bt  # noqa: E402
from paper_conf_date_sunbg021_b200 import _lib as L  # noqa: E402
from synth import KnobSpace, WORKLOADS, make_pool, median_gamma  # noqa: E402

MU = float(np.float32(0.1))
reps = int(sys.argv[1]) if len(sys.argv) > 1 else 20
bad = 0
for N, m in [(1000, 24), (4099, 40), (16384, 64)]:
    _, X = make_pool(KnobSpace(WORKLOADS["resnet18_layer1"], 16), N, 3)
    g = median_gamma(X, 2)
    for name, flags in [("stream", L.BTED_FLAG_NO_SMALL), ("recompute", L.BTED_FLAG_NO_SMALL | L.BTED_FLAG_RECOMPUTE)]:
        ref = None
        for r in range(reps):
            with bt.CandidateSet(X, g, flags=flags) as cs:
                idx, sc = cs.select(m, MU)
            cur = (idx.tolist(), sc.view(np.uint32).tolist())
            if ref is None:
                ref = cur
            elif cur != ref:
                bad += 1
                first = next(t for t in range(m) if cur[0][t] != ref[0][t] or cur[1][t] != ref[1][t])
                print(f"N={N} {name} rep {r}: differs from rep 0 at step {first}")
        print(f"N={N} {name}: {reps} reps done, picks {ref[0][:6]}", flush=True)
print("runs differing:", bad)
