"""K4 completeness on the GPU (refine.cuh header; PAPER.md:138 argmax,
reading A5 lowest index on ties).

Every score unit reports only its best two keys.  When a unit's SECOND key
lies in the near-tie window it may hold a third candidate, and more than 32
candidates never fit the list: such steps are re-scored over ALL unselected
points in fp64 (kFlagFull).  These tests drive exactly those cases on every
engine, at bench-like sizes:

  * K = I (far-apart points, exp underflows to 0 in fp32 and fp64): every
    score ties exactly, so every step has N - t candidates in the window; the
    picks must be 0, 1, ..., m-1 (pin C9 + reading A5);
  * groups of 4 identical consecutive rows (3 twins in the same 32-row unit as
    the pick): exact ties inside one unit, P2 at the fp64 gap GAP_K4 and the
    lowest unselected member of a group always chosen first.
"""
import numpy as np
import pytest

import paper_conf_date_sunbg021_b200 as bt
from paper_conf_date_sunbg021_b200 import _lib as L
from oracle import dense
from synth import KnobSpace, WORKLOADS, make_pool, median_gamma
from tests.parity import check_ted, GAP_K4

pytestmark = pytest.mark.gpu
MU = float(np.float32(0.1))
PACKED = L.BTED_FLAG_NO_SMALL | L.BTED_FLAG_LITERAL
DENSE = L.BTED_FLAG_NO_SMALL | L.BTED_FLAG_DENSE
IMPLICIT = L.BTED_FLAG_NO_SMALL
ENGINES = pytest.mark.parametrize("flags", [IMPLICIT, PACKED, DENSE], ids=["implicit", "packed", "dense"])


@pytest.fixture(scope="module", autouse=True)
def _gpu(need_gpu):
    yield


def far_apart(N):
    """1-D points 100 apart, gamma = 1: K = I exactly in fp32 and in fp64."""
    return (np.arange(N, dtype=np.float32) * 100.0)[:, None]


def grouped_duplicates(n_base, reps=4, seed=61):
    _, Xb = make_pool(KnobSpace(WORKLOADS["resnet18_layer1"], 16), n_base, seed)
    return np.repeat(Xb, reps, axis=0)                    # rows 4g .. 4g+3 identical


def check_group_order(idx, reps=4):
    chosen = set()
    for s in idx.tolist():
        g0 = (s // reps) * reps
        lower = [c for c in range(g0, s) if c not in chosen]
        assert not lower, f"picked {s} while its identical twin {lower[0]} (lower index) was unselected"
        chosen.add(s)


@pytest.mark.parametrize("N", [4096, 16384])
@ENGINES
def test_identity_kernel_bench_size_picks_lowest_indices(N, flags):
    m = 64
    with bt.CandidateSet(far_apart(N), 1.0, flags=flags) as cs:
        L.bted_reset_stats(cs.ctx)
        idx, sc = cs.select(m, MU)
        st = L.bted_get_stats(cs.ctx)
    assert idx.tolist() == list(range(m))                 # C9 + A5
    np.testing.assert_allclose(sc, 1.0 / (1.0 + MU), rtol=1e-6)
    assert st["full_refined_steps"] > 0                   # the candidate lists overflowed and were completed
    assert st["corrected_steps"] == 0


def test_identity_kernel_cluster_engine():
    N, m = 900, 64                                        # the one-kernel cluster TED
    with bt.CandidateSet(far_apart(N), 1.0, flags=L.BTED_FLAG_TIMING) as cs:
        L.bted_reset_stats(cs.ctx)
        idx, _ = cs.select(m, MU)
        st = L.bted_get_stats(cs.ctx)
    assert idx.tolist() == list(range(m))
    assert st["small_teds"] >= 1 and st["full_refined_steps"] > 0


def test_identity_kernel_row_and_tile_shards():
    import torch
    from paper_conf_date_sunbg021_b200.dist import isharded_select_loopback, sharded_select_loopback
    dev = torch.device("cuda", 0)
    st = torch.cuda.Stream(dev)
    X = far_apart(4096)
    for P in (2, 3):
        idx, _ = isharded_select_loopback(X, 1.0, P, 48, MU, dev, st)
        assert idx.tolist() == list(range(48)), f"tile shards P={P}"
        for mode in ("symmetric", "literal"):
            idx, _ = sharded_select_loopback(X, 1.0, P, 48, MU, dev, st, norm_mode=mode)
            assert idx.tolist() == list(range(48)), f"row shards P={P} {mode}"


@ENGINES
def test_grouped_duplicates_within_one_unit(flags):
    X = grouped_duplicates(1024)                          # N = 4096
    g = median_gamma(X, 61)
    m = 96
    with bt.CandidateSet(X, g, flags=flags) as cs:
        L.bted_reset_stats(cs.ctx)
        idx, sc = cs.select(m, MU)
        st = L.bted_get_stats(cs.ctx)
    check_group_order(idx)
    check_ted(idx, sc, dense.ted(X, g, MU, m, forced=idx), f"groups4-{flags}", gap_exact=GAP_K4)
    assert st["full_refined_steps"] > 0
    print(f"groups of 4: refined {st['refined_steps']} (full {st['full_refined_steps']}), "
          f"corrected {st['corrected_steps']}")


def test_grouped_duplicates_cluster_and_shards():
    import torch
    from paper_conf_date_sunbg021_b200.dist import isharded_select_loopback, sharded_select_loopback
    X = grouped_duplicates(200, seed=62)                  # N = 800: cluster kernel
    g = median_gamma(X, 62)
    with bt.CandidateSet(X, g) as cs:
        idx, sc = cs.select(64, MU)
    check_group_order(idx)
    check_ted(idx, sc, dense.ted(X, g, MU, 64, forced=idx), "groups4-cluster", gap_exact=GAP_K4)
    dev = torch.device("cuda", 0)
    st = torch.cuda.Stream(dev)
    X = grouped_duplicates(600, seed=63)                  # N = 2400
    g = median_gamma(X, 63)
    idx, sc = isharded_select_loopback(X, g, 2, 48, MU, dev, st)
    check_group_order(idx)
    check_ted(idx, sc, dense.ted(X, g, MU, 48, forced=idx), "groups4-ishard", gap_exact=GAP_K4)
    idx, sc = sharded_select_loopback(X, g, 3, 48, MU, dev, st)
    check_group_order(idx)
    check_ted(idx, sc, dense.ted(X, g, MU, 48, forced=idx), "groups4-rowshard", gap_exact=GAP_K4)
