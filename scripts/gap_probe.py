"""Where does a BTED call's time go?  Wall time of bted_run_batches vs the
device-timed K1/K2 (BTED_FLAG_TIMING) and K4 refinement counts, with and
without K4 (BTED_FLAG_NO_REFINE).  Usage: python scripts/gap_probe.py [config]"""
import sys
import time

import os
import numpy as np
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import paper_conf_date_sunbg021_b200 as bt
from paper_conf_date_sunbg021_b200 import _lib as L
from synth import config_pool

name = sys.argv[1] if len(sys.argv) > 1 else "vgg16"
X, g, cfg = config_pool(name)
mu = float(np.float32(cfg["mu"]))
for flags, lab in [(L.BTED_FLAG_TIMING, "k4"), (L.BTED_FLAG_TIMING | L.BTED_FLAG_NO_REFINE, "no-k4")]:
    with bt.CandidateSet(X, g, num_batches=cfg["B"], seed=cfg["seed"], flags=flags) as cs:
        cs.run_batches(cfg["M"], cfg["m"], mu)
        L.bted_reset_stats(cs.ctx)
        ts = []
        for _ in range(3):
            t0 = time.perf_counter()
            sel, _ = cs.run_batches(cfg["M"], cfg["m"], mu)
            ts.append(time.perf_counter() - t0)
        st = L.bted_get_stats(cs.ctx)
        print(lab, "wall ms", [round(t * 1e3, 1) for t in ts], "stats", st, "head", list(sel[:4]), flush=True)
