"""One 64-point, 64-pick TED on the cluster kernel (for ncu)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import paper_conf_date_sunbg021_b200 as bt
from synth import KnobSpace, WORKLOADS, make_pool, median_gamma
_, X = make_pool(KnobSpace(WORKLOADS["vgg16_conv1_1"], 16), 64, 7)
g = median_gamma(X, 7)
with bt.CandidateSet(X, g) as cs:
    for _ in range(3):
        cs.select(64, float(np.float32(0.1)))
