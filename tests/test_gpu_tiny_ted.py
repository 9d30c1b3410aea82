"""The one-CTA TED for candidate sets of at most 128 points (small.cuh
ted_tiny_kernel<64 / 128>): the merge TED of Alg. 2 l.6 at the bench's
B m = 64 (and 128 for two batches), and every select / batch TED with N <= 128.  Against the fp64 oracle on
the same seeded inputs (tests/parity.py protocol: P1 on every pick, P2 at the
fp64 gap, with K4 at GAP_K4 where ties are exact)."""
import numpy as np
import pytest

import paper_conf_date_sunbg021_b200 as bt
from paper_conf_date_sunbg021_b200 import _lib as L
from oracle import dense, literal
from oracle.sampling import sample_batches as oracle_sample_batches
from synth import KnobSpace, WORKLOADS, make_pool, uniform_pool, median_gamma
from tests.parity import check_ted, GAP_K4

pytestmark = pytest.mark.gpu
MU = float(np.float32(0.1))


@pytest.fixture(scope="module", autouse=True)
def _gpu(need_gpu):
    yield


def knob(N, d=16, seed=3, wl="resnet18_layer1"):
    _, X = make_pool(KnobSpace(WORKLOADS[wl], d), N, seed)
    return X


@pytest.mark.parametrize("N", [1, 2, 7, 16, 31, 32, 33, 48, 63, 64, 65, 97, 127, 128])
@pytest.mark.parametrize("pool", ["knob", "uniform"])
def test_tiny_ted_matches_oracle(N, pool):
    """Every N of the kernel's range (one and two columns per thread quarter,
    ragged tails), selecting all points (m = N: the merge at B = 1) and a prefix."""
    X = knob(N, seed=N + 11) if pool == "knob" else uniform_pool(N, 16, N + 5)
    g = median_gamma(X, N) if N > 1 else 1.0
    for m in sorted({N, max(1, N // 3)}):
        with bt.CandidateSet(X, g) as cs:
            idx, sc = cs.select(m, MU)
        assert len(set(idx.tolist())) == m
        check_ted(idx, sc, literal.ted(X, g, MU, m, forced=idx), f"tiny-{pool}-{N}-{m}")


@pytest.mark.parametrize("d", [1, 3, 12, 16, 30])
def test_tiny_ted_feature_widths(d):
    X = uniform_pool(57, d, 100 + d)
    g = median_gamma(X, d)
    with bt.CandidateSet(X, g) as cs:
        idx, sc = cs.select(40, MU)
    check_ted(idx, sc, literal.ted(X, g, MU, 40, forced=idx), f"tiny-d{d}")


def test_tiny_ted_linear_kernel():
    X = uniform_pool(50, 8, 9)
    with bt.CandidateSet(X, 1.0, kernel=L.BTED_KERNEL_LINEAR) as cs:
        idx, sc = cs.select(6, MU)
    tr = literal.ted_on_matrix(literal.linear_kernel(X), MU, 6, forced=idx)
    check_ted(idx, sc, tr, "tiny-linear")


@pytest.mark.parametrize("half", [32, 64])
def test_tiny_ted_exact_duplicates_tie_to_lowest_index(half):
    """half points, each twice (rows i and i + half identical): exact fp32 ties on every
    step; K4 re-scores them in fp64 and the lower index of a pair is always taken
    first (reading A5); P2 at the fp64 gap."""
    base = knob(half, seed=91)
    X = np.concatenate([base, base], axis=0)
    n = 2 * half
    g = median_gamma(X, 91)
    with bt.CandidateSet(X, g) as cs:
        L.bted_reset_stats(cs.ctx)
        idx, sc = cs.select(n, MU)
        st = L.bted_get_stats(cs.ctx)
    assert sorted(idx.tolist()) == list(range(n))
    pos = {int(v): t for t, v in enumerate(idx)}
    for i in range(half):
        assert pos[i] < pos[i + half], (i, pos[i], pos[i + half])
    assert st["refined_steps"] > 0
    check_ted(idx, sc, dense.ted(X, g, MU, n, forced=idx), f"tiny-dups-{n}", gap_exact=GAP_K4)


@pytest.mark.parametrize("N", [64, 128])
def test_tiny_ted_far_apart_points_pick_in_index_order(N):
    """K = I (points 100 apart, gamma = 1): every score ties exactly; the picks are
    0, 1, ..., m-1 (pin C9 + reading A5)."""
    X = (np.arange(N, dtype=np.float32) * 100.0).reshape(N, 1)
    with bt.CandidateSet(X, 1.0) as cs:
        idx, _ = cs.select(N, MU)
    assert idx.tolist() == list(range(N))


def test_tiny_ted_batches_and_their_merge():
    """Alg. 2 with batches of M = 50 (each batch TED in the tiny kernel, six
    instances in one launch) and the 120-point merge (tiny kernel, 128-point size)."""
    P, M, B, m, seed = 4000, 50, 6, 20, 31
    X = knob(P, seed=seed)
    g = median_gamma(X, seed)
    with bt.CandidateSet(X, g, num_batches=B, seed=seed) as pool:
        sel, bidx = pool.run_batches(M, m, MU)
        sel2, _ = pool.run_batches(M, m, MU)
    assert np.array_equal(sel, sel2)
    batches = oracle_sample_batches(P, M, B, seed)
    for b in range(B):
        pos = np.searchsorted(batches[b], bidx[b])
        assert np.array_equal(batches[b][pos], bidx[b])
        check_ted(pos, [], literal.ted(X[batches[b]], g, MU, m, forced=pos), f"tiny-batch{b}")
    XU = np.unique(bidx.reshape(-1))
    mpos = np.searchsorted(XU, sel)
    check_ted(mpos, [], literal.ted(X[XU], g, MU, m, forced=mpos), "tiny-batches-merge")


@pytest.mark.parametrize("N", [64, 128])
def test_tiny_ted_is_deterministic_across_calls_and_contexts(N):
    X = knob(N, seed=5)
    g = median_gamma(X, 5)
    with bt.CandidateSet(X, g) as a, bt.CandidateSet(X, g) as b:
        ia, sa = a.select(N, MU)
        ib, sb = b.select(N, MU)
        ia2, sa2 = a.select(N, MU)
    assert np.array_equal(ia, ib) and np.array_equal(sa.view(np.uint32), sb.view(np.uint32))
    assert np.array_equal(ia, ia2) and np.array_equal(sa.view(np.uint32), sa2.view(np.uint32))


def test_tiny_ted_widest_features():
    """d = 64, the widest bted_create accepts, at N = 64 (the features staged in shared memory)."""
    X = uniform_pool(64, 64, 77)
    g = median_gamma(X, 77)
    with bt.CandidateSet(X, g) as cs:
        idx, sc = cs.select(48, MU)
    check_ted(idx, sc, literal.ted(X, g, MU, 48, forced=idx), "tiny-d64")
