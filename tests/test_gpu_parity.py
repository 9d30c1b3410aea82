"""GPU parity: the CUDA path (through the C ABI) against the fp64 oracle on the
same seeded inputs.  Needs a B200 (sm_100a).  Protocol: tests/parity.py."""
import numpy as np
import pytest
from scipy.spatial.distance import cdist

import paper_conf_date_sunbg021_b200 as bt
from paper_conf_date_sunbg021_b200 import _lib as L
from oracle import dense, literal
from oracle.sampling import sample_batches as oracle_sample_batches
from synth import KnobSpace, WORKLOADS, make_pool, uniform_pool, median_gamma, config_pool
from tests.parity import check_ted, ulp32, GAP_K4

pytestmark = pytest.mark.gpu
MU = float(np.float32(0.1))
# engine paths: literal deflation on packed tiles (N4), dense rows, implicit
# deflation (N2, the default), and "auto" (the one-kernel cluster TED of
# small.cuh for N <= ~940, implicit above)
PACKED = L.BTED_FLAG_NO_SMALL | L.BTED_FLAG_LITERAL
DENSE = L.BTED_FLAG_NO_SMALL | L.BTED_FLAG_DENSE
PACKED_TMA = L.BTED_FLAG_NO_SMALL | L.BTED_FLAG_TMA | L.BTED_FLAG_LITERAL
IMPLICIT = L.BTED_FLAG_NO_SMALL                              # the default engine above the cluster TED
LAYOUTS = pytest.mark.parametrize("flags", [PACKED, PACKED_TMA, DENSE, IMPLICIT, 0],
                                  ids=["packed", "packed-tma", "dense", "implicit", "auto"])
LAYOUTS_K = pytest.mark.parametrize("flags", [PACKED, PACKED_TMA, DENSE], ids=["packed", "packed-tma", "dense"])
LAYOUTS_GRAM = pytest.mark.parametrize("flags", [PACKED, PACKED_TMA, DENSE, IMPLICIT],
                                       ids=["packed", "packed-tma", "dense", "implicit"])


@pytest.fixture(scope="module", autouse=True)
def _gpu(need_gpu):
    yield


def knob(N, d=16, seed=3, wl="resnet18_layer1"):
    _, X = make_pool(KnobSpace(WORKLOADS[wl], d), N, seed)
    return X


def ld_of(N):
    return (N + 31) // 32 * 32


# ------------------------------------------------------------------ K1 Gram
@pytest.mark.parametrize("N,d,pool", [(1000, 16, "knob"), (777, 16, "uniform"), (300, 12, "knob"), (515, 30, "uniform")])
def test_implicit_gram_bitwise_equals_k1p(N, d, pool):
    """K1i on CUDA cores (the implicit head's Gram-only kernel, BTED_FLAG_NO_TC_GRAM) writes
    bitwise the tiles K1p writes."""
    X = knob(N, d=d) if pool == "knob" else uniform_pool(N, d, 4)
    g = median_gamma(X, 2)
    with bt.CandidateSet(X, g, flags=IMPLICIT | L.BTED_FLAG_NO_TC_GRAM) as ci, \
            bt.CandidateSet(X, g, flags=PACKED) as cp:
        ci.select(5, MU)
        cp.select(1, MU)
        assert np.array_equal(ci.debug_K(N), cp.debug_K(N))
    with bt.CandidateSet(X, 1.0, kernel=L.BTED_KERNEL_LINEAR, flags=IMPLICIT) as ci, \
            bt.CandidateSet(X, 1.0, kernel=L.BTED_KERNEL_LINEAR, flags=PACKED) as cp:
        ci.select(3, MU)
        cp.select(1, MU)
        assert np.array_equal(ci.debug_K(N), cp.debug_K(N))

@pytest.mark.parametrize("N,pool", [(1000, "knob"), (777, "uniform"), (64, "knob")])
@LAYOUTS_GRAM
def test_gram_entries_bitsymmetric_and_within_ulp_bound(N, pool, flags):
    X = knob(N) if pool == "knob" else uniform_pool(N, 16, 4)
    g = median_gamma(X, 1)
    with bt.CandidateSet(X, g, flags=flags) as cs:
        idx, sc = cs.select(1, MU)
        K = cs.debug_K(N)
    assert K.shape == (N, ld_of(N))
    K32 = K[:, :N].astype(np.float64)
    assert np.all(K[:, N:] == 0.0)                        # zero padding invariant
    assert np.array_equal(K[:, :N], K[:, :N].T)           # bit-symmetric (C1, C6)
    assert np.all(np.diag(K) == 1.0)                      # k(v,v) = 1 exactly
    d2 = cdist(X.astype(np.float64), X.astype(np.float64), "sqeuclidean")
    K64 = np.exp(-float(g) * d2)
    bound = 6.0 * ulp32(K64) * (1.0 + float(g) * d2)
    assert np.all(np.abs(K32 - K64) <= bound), np.max(np.abs(K32 - K64) / ulp32(K64))
    # first pick = argmax of fp64 first scores (C1 + l.3)
    s64 = (K64 * K64).sum(0) / (1.0 + MU)
    assert abs(float(sc[0]) - s64[idx[0]]) <= 1e-5 * s64[idx[0]]


@pytest.mark.parametrize("N,d,pool", [(1000, 16, "knob"), (777, 16, "uniform"), (300, 12, "knob"),
                                      (4099, 16, "knob"), (129, 8, "uniform"), (2000, 16, "knob-dups")])
def test_tensor_core_gram_c1_bound(N, d, pool):
    """K1 on the tensor cores (gram_tc.cuh: centred expansion, bf16x3 tcgen05.mma):
    every entry within pin C1's 6 ulp * (1 + gamma d^2) of fp64, bit-symmetric,
    K_ii = 1, zero padding, exact duplicates give bitwise-equal rows."""
    if pool == "knob-dups":
        X = knob(N // 2, seed=8)
        X = np.concatenate([X, X], axis=0)
    else:
        X = knob(N, d=d) if pool == "knob" else uniform_pool(N, d, 4)
    g = median_gamma(X, 2)
    with bt.CandidateSet(X, g, flags=IMPLICIT) as cs:
        cs.select(2, MU)
        K = cs.debug_K(N)
    K32 = K[:, :N].astype(np.float64)
    assert np.all(K[:, N:] == 0.0)
    assert np.array_equal(K[:, :N], K[:, :N].T)
    assert np.all(np.diag(K) == 1.0)
    d2 = cdist(X.astype(np.float64), X.astype(np.float64), "sqeuclidean")
    K64 = np.exp(-float(g) * d2)
    ratio = np.abs(K32 - K64) / (ulp32(K64) * (1.0 + float(g) * d2))
    print(f"TC Gram N={N} d={d} {pool}: max {ratio.max():.2f} ulp*(1+g d2)")
    assert ratio.max() <= 6.0
    if pool == "knob-dups":                                  # S = D + D' is symmetric bitwise: twins tie
        assert np.array_equal(K[: N // 2, :N], K[N // 2:, :N][:, np.r_[N // 2:N, 0:N // 2]])


def test_tensor_core_gram_guard_falls_back_on_badly_scaled_data():
    """gamma * max |x - c|^2 far above the guard (points 100 apart, gamma = 1):
    the expansion would cancel catastrophically, so the direct-difference kernel
    writes the Gram -- exactly the identity here."""
    N = 3000
    X = (np.arange(N, dtype=np.float32) * 100.0)[:, None]
    with bt.CandidateSet(X, 1.0, flags=IMPLICIT) as cs:
        cs.select(2, MU)
        K = cs.debug_K(N)
    assert np.array_equal(K[:, :N], np.eye(N, dtype=np.float32))


# ------------------------------------------------------------------ K2 step
@LAYOUTS_K
def test_one_deflation_step_vs_fp64_and_selected_column(flags):
    N = 1200
    X = knob(N, seed=9)
    g = median_gamma(X, 2)
    with bt.CandidateSet(X, g, flags=flags) as cs:
        _ = cs.select(1, MU)
        K0 = cs.debug_K(N)[:, :N].astype(np.float64)
        idx, _ = cs.select(2, MU)
        K1 = cs.debug_K(N)[:, :N].astype(np.float64)
        _ = cs.select(9, MU)
        K8 = cs.debug_K(N)
    s = int(idx[0])
    c = K0[s, s] + MU
    prod = np.outer(K0[:, s], K0[s, :]) / c
    ref = K0 - prod                                        # one fp64 step from the GPU's own K0
    tol = 3.0 * ulp32(np.maximum(np.abs(K0), np.abs(prod))) + 1e-30
    assert np.all(np.abs(K1 - ref) <= tol)
    # C5: the selected column scales by mu / (k(s,s) + mu)
    np.testing.assert_allclose(K1[:, s], K0[:, s] * MU / c, rtol=2e-6, atol=1e-30)
    assert np.array_equal(K1, K1.T)
    assert np.array_equal(K8[:, :N], K8[:, :N].T)           # still bit-symmetric after 8 steps


# ------------------------------------------------------------------ TED parity
def k4_on(flags, N):
    """K4 near-tie refinement runs on every single-GPU engine (packed, implicit,
    dense and the small-N cluster kernel) unless BTED_FLAG_NO_REFINE."""
    return not (flags & L.BTED_FLAG_NO_REFINE)


def _ted_parity(X, g, m, label, use_dense=True, flags=0):
    with bt.CandidateSet(X, g, flags=flags) as cs:
        idx, sc = cs.select(m, MU)
        idx2, sc2 = cs.select(m, MU)
    assert np.array_equal(idx, idx2) and np.array_equal(sc.view(np.uint32), sc2.view(np.uint32))  # deterministic
    tr = dense.ted(X, g, MU, m, forced=idx) if use_dense else literal.ted(X, g, MU, m, forced=idx)
    near = check_ted(idx, sc, tr, label, gap_exact=GAP_K4 if k4_on(flags, X.shape[0]) else 1e-6)
    free = dense.ted(X, g, MU, m) if use_dense else literal.ted(X, g, MU, m)
    if min(free.gap) > 1e-6:
        assert idx.tolist() == free.idx, f"{label}: free-running selection differs"
    return near


@LAYOUTS
def test_ted_parity_toy_config(flags):
    X, g, cfg = config_pool("toy")
    _ted_parity(X, g, cfg["m"], "toy", use_dense=False, flags=flags)


@pytest.mark.parametrize("N,pool,m", [(257, "knob", 64), (1000, "uniform", 64), (2049, "knob12", 48),
                                      (4096, "knob", 64), (4096, "uniform", 64)])
@LAYOUTS
def test_ted_parity_multi_tile_ragged(N, pool, m, flags):
    if pool == "knob":
        X = knob(N, seed=N)
    elif pool == "knob12":
        X = knob(N, d=12, seed=N)
    else:
        X = uniform_pool(N, 16, N)
    g = median_gamma(X, N)
    _ted_parity(X, g, m, f"{pool}-{N}", flags=flags)


@LAYOUTS
def test_ted_parity_bench_size_resnet18_batch(flags):
    """The bench workload (resnet18 config: one batch of N = 16384 from the
    2^20-row pool, m = 64), checked at every step against the dense C oracle."""
    X, g, cfg = config_pool("resnet18")
    V = oracle_sample_batches(X.shape[0], cfg["M"], 1, cfg["seed"])[0]
    Xb = X[V]
    with bt.CandidateSet(X, g, num_batches=1, seed=cfg["seed"], flags=flags) as pool:
        sel, bidx = pool.run_batches(cfg["M"], cfg["m"], MU)
    with bt.CandidateSet(Xb, g, flags=flags) as cs:
        idx, sc = cs.select(cfg["m"], MU)
    # the batch TED inside run_batches is the same TED as select on X[V_b]
    assert np.array_equal(V[idx], bidx[0])
    tr = dense.ted(Xb, g, MU, cfg["m"], forced=idx)
    check_ted(idx, sc, tr, "resnet18-16384")
    assert set(sel.tolist()) == set(bidx[0].tolist())      # C10: B = 1 merge keeps the set


# ------------------------------------------------------------------ edge cases
@LAYOUTS
def test_single_point_and_full_permutation(flags):
    X = knob(1)
    with bt.CandidateSet(X, 1.0, flags=flags) as cs:
        idx, sc = cs.select(1, MU)
    assert idx.tolist() == [0] and sc[0] == np.float32(np.float32(1.0) / np.float32(1.0 + MU)) or \
        abs(sc[0] - 1 / (1 + MU)) < 1e-6
    X = knob(100, d=12, seed=5)                              # has exact duplicates
    g = median_gamma(X, 5)
    with bt.CandidateSet(X, g, flags=flags) as cs:
        idx, sc = cs.select(100, MU)
    assert sorted(idx.tolist()) == list(range(100))          # C7: m = N is a permutation


@LAYOUTS
def test_identity_kernel_ties_lowest_index(flags):
    X = (np.arange(40, dtype=np.float32) * 100.0)[:, None]  # K = I exactly in fp32
    with bt.CandidateSet(X, 1.0, flags=flags) as cs:
        idx, sc = cs.select(10, MU)
    assert idx.tolist() == list(range(10))                   # C9 + reading A5
    assert np.all(sc == sc[0])                               # exact ties
    if flags == IMPLICIT:                                    # fp64 recurrence, rounded once to fp32
        np.testing.assert_allclose(sc, 1.0 / (1.0 + MU), rtol=1e-7)
    else:
        assert np.all(sc == np.float32(1.0) / np.float32(np.float32(1.0) + np.float32(MU)))


@LAYOUTS
def test_exact_duplicates_tie_to_lowest_index(flags):
    X = knob(300, seed=2)
    X = np.concatenate([X, X[:50]], axis=0)                  # rows 300..349 duplicate rows 0..49
    g = median_gamma(X, 3)
    with bt.CandidateSet(X, g, flags=flags) as cs:
        idx, sc = cs.select(40, MU)
    for s in idx:
        assert s < 300 or (s - 300) in idx[: list(idx).index(s)], "duplicate chosen before its twin"
    tr = dense.ted(X, g, MU, 40, forced=idx)
    check_ted(idx, sc, tr, "dups")


@LAYOUTS_K
def test_linear_kernel_closed_form_c8(flags):
    rng = np.random.default_rng(8)
    X = (rng.standard_normal((300, 6)) * 0.5).astype(np.float32)
    with bt.CandidateSet(X, 1.0, kernel=L.BTED_KERNEL_LINEAR, flags=flags) as cs:
        idx, sc = cs.select(6, MU)
        K5 = cs.debug_K(300)[:, :300].astype(np.float64)
    Xd = X.astype(np.float64)
    XS = Xd[idx[:5]]
    ref = MU * Xd @ np.linalg.inv(MU * np.eye(6) + XS.T @ XS) @ Xd.T
    assert np.max(np.abs(K5 - ref)) < 2e-5 * np.abs(Xd @ Xd.T).max()
    tr = literal.ted_on_matrix(literal.linear_kernel(X), MU, 6, forced=idx)
    check_ted(idx, sc, tr, "linear")


def test_invalid_arguments_fail_loudly():
    X = knob(50)
    with bt.CandidateSet(X, 0.5) as cs:
        for m, mu in [(0, MU), (51, MU), (5, 0.0), (5, float("nan"))]:
            with pytest.raises(bt.BtedError) as e:
                cs.select(m, mu)
            assert e.value.status == 1
    bad = X.copy()
    bad[3, 2] = np.nan
    with pytest.raises(bt.BtedError):
        bt.CandidateSet(bad, 0.5)
    with pytest.raises(bt.BtedError):
        bt.CandidateSet(X, -1.0)


# ------------------------------------------------------------------ Alg. 2
@pytest.mark.parametrize("P,M,B,seed", [(1 << 20, 16384, 2, 5), (777, 777, 2, 1), (1000, 1, 3, 9),
                                        (50000, 2048, 4, 3)])
def test_sampling_bit_exact_vs_oracle_sampler(P, M, B, seed):
    gpu = bt.bted_sample_batches(P, M, B, seed)
    ref = oracle_sample_batches(P, M, B, seed)
    assert np.array_equal(gpu, ref)


def _positions(V, pool_idx):
    pos = np.searchsorted(V, pool_idx)
    assert np.array_equal(V[pos], pool_idx)
    return pos


@LAYOUTS
def test_bted_parity_vs_oracle(flags):
    P, M, B, m, seed = 60000, 2048, 4, 32, 3
    space = KnobSpace(WORKLOADS["vgg16_conv1_1"], 16)
    _, X = make_pool(space, P, 77)
    g = median_gamma(X, 77)
    with bt.CandidateSet(X, g, num_batches=B, seed=seed, flags=flags) as pool:
        sel, bidx = pool.run_batches(M, m, MU)
    batches = oracle_sample_batches(P, M, B, seed)
    for b in range(B):
        Vb = batches[b]
        pos = _positions(Vb, bidx[b])
        tr = dense.ted(X[Vb], g, MU, m, forced=pos)
        check_ted(pos, [], tr, f"batch{b}")
    XU = np.unique(bidx)                                     # Alg. 2 l.5
    assert set(sel.tolist()) <= set(XU.tolist()) and len(sel) == min(m, len(XU))
    mpos = _positions(XU, sel)
    trm = literal.ted(X[XU], g, MU, len(sel), forced=mpos)   # l.6 on a fresh Gram of X_U
    check_ted(mpos, [], trm, "merge")


@LAYOUTS
def test_round_robin_batches_then_merge_equals_run_batches(flags):
    P, M, B, m, seed = 30000, 1024, 5, 16, 11
    X = knob(P, seed=4)
    g = median_gamma(X, 4)
    with bt.CandidateSet(X, g, num_batches=B, seed=seed, flags=flags) as pool:
        sel, bidx = pool.run_batches(M, m, MU)
        w0 = np.empty(3 * m, np.int64)
        w1 = np.full(3 * m, -1, np.int64)                    # rank 1 has 2 batches: padded like an all-gather
        pool.batch_teds(M, m, MU, 0, 2, w0)
        pool.batch_teds(M, m, MU, 1, 2, w1)
        assert np.array_equal(w0.reshape(3, m), bidx[0::2]) and np.array_equal(w1[: 2 * m].reshape(2, m), bidx[1::2])
        sel2 = pool.merge(np.concatenate([w0, w1]), 6 * m, m, MU)
    assert np.array_equal(sel, sel2)


def test_merge_smaller_than_m():
    X = knob(500, seed=6)
    g = median_gamma(X, 6)
    with bt.CandidateSet(X, g) as pool:
        out = pool.merge(np.array([5, 9, 5, 100, -1, 9]), 6, 8, MU)
    assert sorted(out.tolist()) == [5, 9, 100]               # A12: select all of X_U


# ------------------------------------------------------------------ sharded
@pytest.mark.parametrize("N,P", [(3000, 2), (3001, 3), (1024, 4)])
def test_row_sharded_loopback_bit_identical(N, P):
    import torch
    from paper_conf_date_sunbg021_b200.dist import sharded_select_loopback
    X = knob(N, seed=N + P)
    g = median_gamma(X, P)
    with bt.CandidateSet(X, g, flags=DENSE) as cs:     # shards are dense
        idx, sc = cs.select(24, MU)
    dev = torch.device("cuda", 0)
    st = torch.cuda.Stream(dev)
    sidx, ssc = sharded_select_loopback(X, g, P, 24, MU, dev, st)
    assert np.array_equal(sidx, idx)
    assert np.array_equal(ssc.view(np.uint32), sc.view(np.uint32))


@pytest.mark.parametrize("N,P", [(3001, 1), (3001, 3), (1024, 4)])
def test_row_sharded_literal_column_norms_vs_oracle(N, P):
    """norm_mode='literal' (north_star: all-reduce of partial column norms): the
    band values are those of the symmetric mode; the column-norm scores pass
    P1/P2 against the fp64 oracle along the GPU's picks."""
    import torch
    from paper_conf_date_sunbg021_b200.dist import sharded_select_loopback
    X = knob(N, seed=N + 7 * P)
    g = median_gamma(X, P)
    dev = torch.device("cuda", 0)
    st = torch.cuda.Stream(dev)
    m = 24
    lidx, lsc = sharded_select_loopback(X, g, P, m, MU, dev, st, norm_mode="literal")
    tr = literal.ted(X, g, MU, m, forced=lidx.tolist())
    check_ted(lidx, lsc, tr, f"literal-colnorm N={N} P={P}", gap_exact=GAP_K4)
    sidx, ssc = sharded_select_loopback(X, g, P, m, MU, dev, st)
    assert len(set(lidx.tolist())) == m
    np.testing.assert_allclose(lsc, ssc, rtol=1e-5)         # same numbers up to rounding order


@pytest.mark.parametrize("N,P,d", [(3001, 1, 16), (3001, 2, 16), (2500, 3, 12), (1100, 5, 16), (4096, 4, 30)])
def test_tile_sharded_implicit_loopback_vs_oracle(N, P, d):
    """ShardedImplicitTed (Gram tiles k = r mod P, one q all-reduce per step)
    with P logical shards on one GPU: P1/P2 against the fp64 oracle along its
    picks, the same picks as the single-GPU implicit engine wherever the
    oracle's gap is clear, and scores within 1e-5 of it."""
    import torch
    from paper_conf_date_sunbg021_b200.dist import isharded_select_loopback
    X = knob(N, d=d, seed=N + P) if d != 30 else uniform_pool(N, d, P)
    g = median_gamma(X, P)
    dev = torch.device("cuda", 0)
    st = torch.cuda.Stream(dev)
    m = 40
    idx, sc = isharded_select_loopback(X, g, P, m, MU, dev, st)
    assert len(set(idx.tolist())) == m
    tr = dense.ted(X, g, MU, m, forced=idx)
    check_ted(idx, sc, tr, f"ishard N={N} P={P}")
    with bt.CandidateSet(X, g, flags=IMPLICIT | L.BTED_FLAG_NO_REFINE) as cs:
        i1, s1 = cs.select(m, MU)
    k = int(np.argmax(i1 != idx)) if not np.array_equal(i1, idx) else m
    assert k == m or tr.gap[k] <= 1e-5, (k, tr.gap[k])
    np.testing.assert_allclose(sc[:k], s1[:k], rtol=1e-5)


@pytest.mark.parametrize("P", [2, 3])
def test_tile_sharded_implicit_k4_exact_ties(P):
    """Exact duplicates: the shards' q sums are not bitwise equal for the two
    copies, so the fp32 order of tied scores is rounding; K4 (bted_ishard_refine,
    fp64 from the replicated features) must still give the lowest index and
    P2 at the fp64 gap GAP_K4."""
    import torch
    from paper_conf_date_sunbg021_b200.dist import isharded_select_loopback
    X = knob(2500, seed=43)
    X = np.concatenate([X, X[::5]], axis=0)                  # 500 exact duplicate pairs
    g = median_gamma(X, 43)
    dev = torch.device("cuda", 0)
    st = torch.cuda.Stream(dev)
    st_k4 = {}
    idx, sc = isharded_select_loopback(X, g, P, 64, MU, dev, st, stats=st_k4)
    assert st_k4["refined_steps"] > 0                        # the tied steps went through K4
    check_ted(idx, sc, dense.ted(X, g, MU, 64, forced=idx), f"ishard-k4 P={P}", gap_exact=GAP_K4)
    print(f"ishard K4 P={P}: refined {st_k4['refined_steps']}, corrected {st_k4['corrected_steps']}")


@pytest.mark.parametrize("norm_mode", ["symmetric", "literal"])
@pytest.mark.parametrize("P", [1, 2, 3])
def test_row_sharded_k4_exact_ties(P, norm_mode):
    """Row bands (symmetric mode, and the literal column-norm ablation) with K4:
    near-tie candidates of every band, gathered over the shards, re-scored in
    fp64; P2 at the fp64 gap."""
    import torch
    from paper_conf_date_sunbg021_b200.dist import sharded_select_loopback
    X = uniform_pool(1800, 8, 53)
    Xn = X[::4].copy()
    Xn[:, 1] += np.float32(2e-4)                             # near duplicates: fp64 gaps below fp32 noise
    X = np.concatenate([X, Xn], axis=0)
    g = median_gamma(X, 53)
    dev = torch.device("cuda", 0)
    st = torch.cuda.Stream(dev)
    k4 = {}
    idx, sc = sharded_select_loopback(X, g, P, 200, MU, dev, st, norm_mode=norm_mode, stats=k4)
    assert k4["refined_steps"] > 0
    check_ted(idx, sc, dense.ted(X, g, MU, 200, forced=idx), f"rowshard-k4-{norm_mode} P={P}", gap_exact=GAP_K4)
    print(f"row-shard K4 {norm_mode} P={P}: refined {k4['refined_steps']}, corrected {k4['corrected_steps']}")


def test_launch_counter_counts_kernels():
    X = knob(300)
    before = bt.bted_kernel_launches()
    with bt.CandidateSet(X, 0.3, flags=DENSE) as cs:
        cs.select(10, MU)
    assert bt.bted_kernel_launches() - before == 1 + 11 + 1  # finite check + transpose + K1 + 9 x K2 + K4 check
    before = bt.bted_kernel_launches()
    with bt.CandidateSet(X, 0.3, flags=PACKED) as cs:
        cs.select(10, MU)
    assert bt.bted_kernel_launches() - before == 1 + 20 + 1  # finite check + K1p + fin + 9 x (K2p + fin) + K4 check
    before = bt.bted_kernel_launches()
    with bt.CandidateSet(X, 0.3, flags=PACKED_TMA) as cs:
        cs.select(10, MU)
    assert bt.bted_kernel_launches() - before == 1 + 20 + 1  # finite check + K1p + fin + 9 x (TMA K2p + fin) + K4
    before = bt.bted_kernel_launches()
    with bt.CandidateSet(X, 0.3, flags=IMPLICIT | L.BTED_FLAG_PERSISTENT_LOOP) as cs:
        cs.select(10, MU)
    assert bt.bted_kernel_launches() - before == 1 + 4 + 1   # finite check + K1p + norm pass + fin + the loop kernel + K4
    before = bt.bted_kernel_launches()
    with bt.CandidateSet(X, 0.3, flags=IMPLICIT) as cs:
        cs.select(10, MU)
    assert bt.bted_kernel_launches() - before == 1 + 30 + 1  # finite check + K1p + norm pass + fin + 9 x (ell + q + fin) + K4
    before = bt.bted_kernel_launches()
    with bt.CandidateSet(X, 0.3) as cs:
        cs.select(10, MU)
    assert bt.bted_kernel_launches() - before == 1 + 1 + 1   # finite check + the whole TED in one cluster kernel + K4 check


# ------------------------------------------------------------------ packed vs dense layout
@pytest.mark.parametrize("N,d,m", [(1000, 16, 40), (4099, 16, 64), (300, 12, 300), (129, 30, 20)])
def test_packed_layout_matches_dense(N, d, m):
    """Packed-symmetric storage (N4) computes every element of K bitwise like
    the dense layout; only the norm summation order differs."""
    X = knob(N, d=16, seed=N)[:, :d] if d <= 16 else uniform_pool(N, d, N)
    g = median_gamma(X, d)
    with bt.CandidateSet(X, g, flags=DENSE) as cd, bt.CandidateSet(X, g, flags=PACKED) as cp, \
            bt.CandidateSet(X, g, flags=PACKED_TMA) as ct, bt.CandidateSet(X, g, flags=IMPLICIT) as ci:
        i_i, s_i = ci.select(m, MU)
        check_ted(i_i, s_i, dense.ted(X, g, MU, m, forced=i_i), f"implicit-{N}")
        i_d, s_d = cd.select(m, MU)
        i_p, s_p = cp.select(m, MU)
        i_t, s_t = ct.select(m, MU)
        assert np.array_equal(i_t, i_p) and np.array_equal(s_t.view(np.uint32), s_p.view(np.uint32))
        assert np.array_equal(ct.debug_K(N), cp.debug_K(N))       # TMA and LDG variants: same bits
        tr = dense.ted(X, g, MU, m, forced=i_p)
        check_ted(i_p, s_p, tr, f"packed-{N}")
        if np.array_equal(i_d, i_p):
            np.testing.assert_allclose(s_p, s_d, rtol=2e-6)
            Kd, Kp = cd.debug_K(N), cp.debug_K(N)
            assert np.array_equal(Kd[:, :N], Kp[:, :N])      # same pivots -> bitwise equal K
            assert np.all(Kp[:, N:] == 0)
        else:                                                  # only legitimate near-ties may differ
            k = int(np.argmax(i_d != i_p))
            assert tr.gap[k] <= 1e-5


# ------------------------------------------------------------------ paper-scale (N3) and the cluster TED
def test_paper_scale_bted_vs_oracle():
    """The paper's own BTED workload: B = 10 batches of M = 500
    points, m = 64, union of <= 640 points; batch TEDs and the merge run as
    cluster kernels (small.cuh)."""
    X, g, cfg = config_pool("paper")
    B, M, m = cfg["B"], cfg["M"], cfg["m"]
    with bt.CandidateSet(X, g, num_batches=B, seed=cfg["seed"]) as pool:
        before = bt.bted_kernel_launches()
        sel, bidx = pool.run_batches(M, m, MU)
        launched = bt.bted_kernel_launches() - before
    batches = oracle_sample_batches(X.shape[0], M, B, cfg["seed"])
    for b in range(B):
        pos = _positions(batches[b], bidx[b])
        check_ted(pos, [], literal.ted(X[batches[b]], g, MU, m, forced=pos), f"paper-batch{b}")
    XU = np.unique(bidx)
    assert len(XU) == len(set(bidx.ravel().tolist()))
    mpos = _positions(XU, sel)
    check_ted(mpos, [], literal.ted(X[XU], g, MU, len(sel), forced=mpos), "paper-merge")
    # one cluster launch for all 10 batch TEDs + one for the merge (+ sampling/gather/union kernels)
    assert launched < 60


@pytest.mark.parametrize("N,m", [(1000, 64), (4099, 64), (300, 256), (2000, 200)])
def test_implicit_deflation_matches_oracle(N, m):
    """N2: K read-only + fp64 factor recurrences -> same picks as the oracle."""
    X = knob(N, seed=N + 11)
    g = median_gamma(X, N)
    with bt.CandidateSet(X, g, flags=IMPLICIT) as cs:
        idx, sc = cs.select(m, MU)
        idx2, sc2 = cs.select(m, MU)
    assert np.array_equal(idx, idx2) and np.array_equal(sc.view(np.uint32), sc2.view(np.uint32))
    tr = dense.ted(X, g, MU, m, forced=idx)
    check_ted(idx, sc, tr, f"implicit-{N}")


@pytest.mark.parametrize("N,m", [(1000, 64), (4099, 40), (16384, 64), (1500, 256)])
def test_persistent_loop_equals_step_kernels(N, m):
    """The one-launch persistent loop (grid barriers) runs the same arithmetic in
    the same order as the three-kernels-per-step loop: identical picks and score bits."""
    X = knob(N, seed=N + 5) if N != 1500 else uniform_pool(N, 8, 77)
    g = median_gamma(X, N)
    with bt.CandidateSet(X, g, flags=IMPLICIT | L.BTED_FLAG_PERSISTENT_LOOP) as a, \
            bt.CandidateSet(X, g, flags=IMPLICIT) as b:
        ia, sa = a.select(m, MU)
        ib, sb = b.select(m, MU)
        ia2, sa2 = a.select(m, MU)
    assert np.array_equal(ia, ib) and np.array_equal(sa.view(np.uint32), sb.view(np.uint32))
    assert np.array_equal(ia, ia2) and np.array_equal(sa.view(np.uint32), sa2.view(np.uint32))


@pytest.mark.parametrize("N", [1, 5, 64, 230, 231, 500, 640, 777, 940])
def test_cluster_ted_matches_oracle_across_cluster_sizes(N):
    X = knob(N, seed=N + 7)
    g = median_gamma(X, N) if N > 1 else 1.0
    m = min(N, 48)
    with bt.CandidateSet(X, g) as cs:
        idx, sc = cs.select(m, MU)
    tr = literal.ted(X, g, MU, m, forced=idx)
    check_ted(idx, sc, tr, f"cluster-{N}")


# ------------------------------------------------------------------ full size: oversized batch
def test_oversized_65536_sampled_against_closed_form():
    """BASELINE config 'oversized': one TED on N = 65536 (d = 16, m = 64) in
    the default (packed) layout, checked on sampled outputs one by one with
    the matrix-free fp64 oracle (oracle/closed_form.py): P1 at EVERY step
    (the pick's score vs its fp64 score given the same history), and at four
    steps no sampled candidate beats the pick by more than the 1e-6 gap rule."""
    from oracle.closed_form import ClosedForm
    X, g, cfg = config_pool("oversized")
    V = oracle_sample_batches(X.shape[0], cfg["M"], 1, cfg["seed"])[0]
    Xb = X[V]
    m = cfg["m"]
    with bt.CandidateSet(Xb, g) as cs:
        idx, sc = cs.select(m, MU)
    assert len(set(idx.tolist())) == m
    cf = ClosedForm(Xb, g, MU)
    rng = np.random.default_rng(65536)
    for t in range(m):
        s64 = cf.scores([idx[t]])[0]
        assert abs(float(sc[t]) - s64) <= 1e-5 * s64, (t, float(sc[t]), s64)          # P1
        if t in (0, 1, 31, m - 1):
            cand = rng.choice(cfg["M"], 384, replace=False)
            cand = np.array([c for c in cand if c not in set(idx[:t].tolist())])
            other = cf.scores(cand)
            assert other.max() <= s64 * (1 + 1e-6), (t, other.max(), s64)             # sampled P2
        cf.add(idx[t])


def test_update_replaces_features_and_validates_on_device():
    X1, X2 = knob(3000, seed=1), knob(3000, seed=2)
    g = median_gamma(X1, 1)
    with bt.CandidateSet(X2, g, num_batches=2, seed=4) as ref:
        want = ref.run_batches(1000, 16, MU)[0]
    with bt.CandidateSet(X1, g, num_batches=2, seed=4) as cs:
        first = cs.run_batches(1000, 16, MU)[0]
        L.bted_update(cs.ctx, X2)
        assert np.array_equal(cs.run_batches(1000, 16, MU)[0], want)
        bad = X2.copy()
        bad[7, 3] = np.inf
        L.bted_update(cs.ctx, bad)
        with pytest.raises(bt.BtedError) as e:
            cs.run_batches(1000, 16, MU)
        assert e.value.status == 1 and "non-finite" in str(e.value)
        L.bted_update(cs.ctx, X1)                                   # recovers
        assert np.array_equal(cs.run_batches(1000, 16, MU)[0], first)


@pytest.mark.parametrize("flags", [IMPLICIT, PACKED, DENSE], ids=["implicit", "packed", "dense"])
def test_subnormal_and_underflowing_kernel_values(flags):
    """gamma large enough that many K_ij are fp32 subnormals or underflow to 0
    (exercises the implicit tile pass's conversion fallback)."""
    X = uniform_pool(700, 16, 70)
    g = 30.0
    with bt.CandidateSet(X, g, flags=flags) as cs:
        idx, sc = cs.select(32, MU)
    tr = dense.ted(X, g, MU, 32, forced=idx)
    check_ted(idx, sc, tr, f"subnormal-{flags}")


# ------------------------------------------------------------------ K4 near-tie refinement
def test_k4_resolves_exact_ties_and_counts():
    """Exact duplicates make exact ties: with K4 the tied steps are re-scored in
    fp64 and resolved to the lowest index; P2 then holds at the fp64 level."""
    X = knob(3000, seed=41)
    X = np.concatenate([X, X[::7]], axis=0)                  # ~430 exact duplicate pairs
    g = median_gamma(X, 41)
    with bt.CandidateSet(X, g, flags=PACKED) as cs:
        L.bted_reset_stats(cs.ctx)
        idx, sc = cs.select(96, MU)
        st = L.bted_get_stats(cs.ctx)
    tr = dense.ted(X, g, MU, 96, forced=idx)
    check_ted(idx, sc, tr, "k4-dups", gap_exact=GAP_K4)


@pytest.mark.parametrize("flags", [PACKED, IMPLICIT, DENSE], ids=["packed", "implicit", "dense"])
def test_k4_strict_parity_on_long_selections(flags):
    """Long selections (small late scores, many near ties): every pick equals
    the fp64 oracle's argmax wherever the oracle's gap exceeds 1e-9."""
    total_refined = total_corrected = 0
    for seed in range(6):
        X = uniform_pool(1500, 8, 900 + seed)
        g = median_gamma(X, seed)
        with bt.CandidateSet(X, g, flags=flags) as cs:
            L.bted_reset_stats(cs.ctx)
            idx, sc = cs.select(300, MU)
            st = L.bted_get_stats(cs.ctx)
        total_refined += st["refined_steps"]
        total_corrected += st["corrected_steps"]
        tr = dense.ted(X, g, MU, 300, forced=idx)
        check_ted(idx, sc, tr, f"k4-long-{seed}", gap_exact=GAP_K4)
    print(f"K4: refined {total_refined} steps, corrected {total_corrected}")


@pytest.mark.parametrize("flags", [PACKED, IMPLICIT, DENSE], ids=["packed", "implicit", "dense"])
def test_k4_in_batches_matches_oracle_strictly(flags):
    """Alg. 2 batch TEDs keep their own K4 state (keys, flags, candidates per
    batch); the flagged steps are refined after all batches without re-running
    them, and every batch still meets P2 at the fp64 gap GAP_K4."""
    X = uniform_pool(5000, 8, 5)
    X = np.concatenate([X, X[::5]], axis=0)                  # exact duplicates: exact ties to refine
    P, M, B, m, seed = X.shape[0], 1500, 4, 200, 17
    g = median_gamma(X, 5)
    with bt.CandidateSet(X, g, num_batches=B, seed=seed, flags=flags) as pool:
        L.bted_reset_stats(pool.ctx)
        launches = bt.bted_kernel_launches()
        sel, bidx = pool.run_batches(M, m, MU)
        launches = bt.bted_kernel_launches() - launches
        st = L.bted_get_stats(pool.ctx)
        sel2, bidx2 = pool.run_batches(M, m, MU)              # deterministic
    assert np.array_equal(sel, sel2) and np.array_equal(bidx, bidx2)
    assert st["refined_steps"] > 0                           # the refinement path ran
    batches = oracle_sample_batches(P, M, B, seed)
    for b in range(B):
        pos = _positions(batches[b], bidx[b])
        check_ted(pos, [], dense.ted(X[batches[b]], g, MU, m, forced=pos), f"k4-batch{b}", gap_exact=GAP_K4)
    print(f"K4 in batches: refined {st['refined_steps']}, corrected {st['corrected_steps']}, launches {launches}")


def test_k4_cluster_kernel_exact_ties():
    """K4 on the one-kernel cluster TED (small candidate sets: merges, paper-scale
    batches): exact duplicates give exact fp32 ties; every flagged step is
    re-scored in fp64 and P2 holds at the fp64 gap, for a small select, the
    paper-scale batches and their merge."""
    X = knob(600, seed=47)
    X = np.concatenate([X, X[::3]], axis=0)                  # 800 points, 200 exact duplicate pairs
    g = median_gamma(X, 47)
    with bt.CandidateSet(X, g) as cs:                          # N = 800: the cluster kernel
        L.bted_reset_stats(cs.ctx)
        idx, sc = cs.select(96, MU)
        st = L.bted_get_stats(cs.ctx)
    assert st["refined_steps"] > 0
    check_ted(idx, sc, dense.ted(X, g, MU, 96, forced=idx), "k4-cluster", gap_exact=GAP_K4)
    P, M, B, m, seed = X.shape[0], 300, 4, 64, 23
    with bt.CandidateSet(X, g, num_batches=B, seed=seed) as pool:     # batches and merge in cluster kernels
        sel, bidx = pool.run_batches(M, m, MU)
        sel2, _ = pool.run_batches(M, m, MU)
    assert np.array_equal(sel, sel2)
    batches = oracle_sample_batches(P, M, B, seed)
    for b in range(B):
        pos = _positions(batches[b], bidx[b])
        check_ted(pos, [], dense.ted(X[batches[b]], g, MU, m, forced=pos), f"k4-cluster-batch{b}", gap_exact=GAP_K4)
    XU = np.unique(bidx.reshape(-1))
    mpos = _positions(XU, sel)
    check_ted(mpos, [], dense.ted(X[XU], g, MU, m, forced=mpos), "k4-cluster-merge", gap_exact=GAP_K4)


def test_k4_cluster_kernel_long_selections():
    """Long selections on the cluster kernel (small N, late steps with small
    scores and many near ties): P2 at the fp64 gap on every seed; the forced
    re-launch path runs whenever a refined pick changes."""
    total_refined = total_corrected = 0
    for seed in range(6):
        X = uniform_pool(720, 8, 700 + seed)
        Xn = X[::4].copy()
        Xn[:, seed % 8] += np.float32(2e-4)                  # near duplicates: fp64 gaps far below fp32 noise
        X = np.concatenate([X, Xn], axis=0)
        g = median_gamma(X, seed)
        with bt.CandidateSet(X, g) as cs:
            L.bted_reset_stats(cs.ctx)
            idx, sc = cs.select(300, MU)
            st = L.bted_get_stats(cs.ctx)
        total_refined += st["refined_steps"]
        total_corrected += st["corrected_steps"]
        check_ted(idx, sc, dense.ted(X, g, MU, 300, forced=idx), f"k4-cluster-long-{seed}", gap_exact=GAP_K4)
    print(f"cluster K4: refined {total_refined} steps, corrected {total_corrected}")
    assert total_refined > 0 and total_corrected > 0         # the forced re-launch path ran (deterministic)


def test_large_131072_sampled_against_closed_form():
    """one un-batched TED on N = 131072 (K = 34 GB per packed
    buffer), P1 at every step and sampled P2, as for 'oversized'."""
    from oracle.closed_form import ClosedForm
    X, g, cfg = config_pool("large")
    V = oracle_sample_batches(X.shape[0], cfg["M"], 1, cfg["seed"])[0]
    Xb = X[V]
    m = cfg["m"]
    with bt.CandidateSet(Xb, g) as cs:
        idx, sc = cs.select(m, MU)
    assert len(set(idx.tolist())) == m
    cf = ClosedForm(Xb, g, MU)
    rng = np.random.default_rng(131072)
    for t in range(m):
        s64 = cf.scores([idx[t]])[0]
        assert abs(float(sc[t]) - s64) <= 1e-5 * s64, (t, float(sc[t]), s64)
        if t in (0, 32, m - 1):
            cand = rng.choice(cfg["M"], 192, replace=False)
            cand = np.array([c for c in cand if c not in set(idx[:t].tolist())])
            assert cf.scores(cand).max() <= s64 * (1 + 1e-6)
        cf.add(idx[t])


@pytest.mark.parametrize("B", [64, 70], ids=["one-cta-union-4096", "cub-union-4480"])
def test_union_of_many_batches_both_paths(B):
    """Alg. 2 l.5 with B * m winners at the one-CTA union's limit (4096) and above
    it (the CUB sort + unique path): X_U is exactly the sorted unique winners and
    the merge TED passes P2 against the oracle on a fresh Gram of X_U."""
    P, M, m, seed = 20000, 256, 64, 31
    X = knob(P, seed=12)
    g = median_gamma(X, 12)
    with bt.CandidateSet(X, g, num_batches=B, seed=seed) as pool:
        sel, bidx = pool.run_batches(M, m, MU)
    XU = np.unique(bidx.reshape(-1))
    assert len(sel) == m and set(sel.tolist()) <= set(XU.tolist())
    mpos = _positions(XU, sel)
    check_ted(mpos, [], dense.ted(X[XU], g, MU, m, forced=mpos), f"union-{B}", gap_exact=GAP_K4)
