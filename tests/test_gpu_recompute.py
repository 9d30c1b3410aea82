"""The recomputing K.l pass (csrc/rc_pass.cuh): every greedy step rebuilds the
Gram tiles on the tensor cores instead of streaming the stored Gram from HBM.
It must be the SAME computation -- the same K entries (the MMA results do not
depend on an operand's position, the epilogue is the stored Gram's function)
and the same fp64 consumer -- so picks and fp32 scores are bitwise those of the
streaming pass (the default), and both pass the oracle protocol."""
import numpy as np
import pytest

import paper_conf_date_sunbg021_b200 as bt
from paper_conf_date_sunbg021_b200 import _lib as L
from oracle import dense
from synth import KnobSpace, WORKLOADS, make_pool, uniform_pool, median_gamma
from tests.parity import check_ted, GAP_K4

pytestmark = pytest.mark.gpu
MU = float(np.float32(0.1))
STREAM = L.BTED_FLAG_NO_SMALL                               # the default implicit engine
IMPLICIT = STREAM | L.BTED_FLAG_RECOMPUTE                   # ... with the recomputing K.l pass


def knob(N, d=16, seed=3, wl="resnet18_layer1"):
    _, X = make_pool(KnobSpace(WORKLOADS[wl], d), N, seed)
    return X


def both(X, g, m, extra=0):
    with bt.CandidateSet(X, g, flags=IMPLICIT | extra) as cs:
        a = cs.select(m, MU)
    with bt.CandidateSet(X, g, flags=STREAM | extra) as cs:
        b = cs.select(m, MU)
    return a, b


@pytest.mark.parametrize("N,pool,m", [(1000, "knob", 24), (4099, "knob", 40), (2048, "uniform", 32),
                                      (16384, "knob", 64), (12345, "dups", 48), (129, "knob", 8)])
def test_recompute_pass_bitwise_equals_streaming_pass(need_gpu, N, pool, m):
    if pool == "dups":                                        # exact duplicates: ties to the lowest index
        X = knob(N // 2 + 1, seed=11)
        X = np.concatenate([X, X], axis=0)[:N]
    elif pool == "uniform":
        X = uniform_pool(N, 16, 4)
    else:
        X = knob(N)
    g = median_gamma(X, 2)
    (ia, sa), (ib, sb) = both(X, g, m)
    assert np.array_equal(ia, ib)
    assert np.array_equal(sa.view(np.uint32), sb.view(np.uint32))


def test_recompute_pass_oracle_protocol(need_gpu):
    """P1/P2 (teacher-forced, every step, K4 gap) against the dense fp64 oracle."""
    X = knob(3000, seed=21)
    g = median_gamma(X, 21)
    with bt.CandidateSet(X, g, flags=IMPLICIT) as cs:
        idx, sc = cs.select(48, MU)
    tr = dense.ted(X, g, MU, 48, forced=idx)
    check_ted(idx, sc, tr, "recompute-3000", gap_exact=GAP_K4)


def test_recompute_guard_fallback_streams_the_stored_gram(need_gpu):
    """Badly scaled data (the tensor-core guard fails): the pass streams the
    direct-form Gram instead -- the identity here, so picks 0, 1, 2, ..."""
    N = 3000
    X = (np.arange(N, dtype=np.float32) * 100.0)[:, None]
    with bt.CandidateSet(X, 1.0, flags=IMPLICIT) as cs:
        idx, _ = cs.select(16, MU)
    assert list(idx) == list(range(16))


def test_recompute_in_batches_bitwise(need_gpu):
    _, P = make_pool(KnobSpace(WORKLOADS["resnet18_layer1"], 16), 60000, 7)
    g = median_gamma(P, 7)
    with bt.CandidateSet(P, g, num_batches=3, seed=2, flags=L.BTED_FLAG_RECOMPUTE) as pool:
        a, _ = pool.run_batches(4096, 32, MU)
    with bt.CandidateSet(P, g, num_batches=3, seed=2) as pool:
        b, _ = pool.run_batches(4096, 32, MU)
    assert np.array_equal(a, b)
