"""Cluster-TED timing split (Gram phase vs greedy steps): select(1) vs select(m) on N points."""
import os
import sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import paper_conf_date_sunbg021_b200 as bt
from synth import KnobSpace, WORKLOADS, make_pool, median_gamma

for N in (64, 500, 640):
    _, X = make_pool(KnobSpace(WORKLOADS["vgg16_conv1_1"], 16), N, 7)
    g = median_gamma(X, 7)
    with bt.CandidateSet(X, g) as cs:
        for m in (1, 64):
            for _ in range(3):
                cs.select(m, float(np.float32(0.1)))
