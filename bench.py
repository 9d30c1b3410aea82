#!/usr/bin/env python
"""Benchmark of the BTED hot path (BASELINE.json metric) on B200.

  python bench.py [--gpus N] [--steps K] [--warmup W] [--config resnet18] [--impl ours|reference]

A step = one pass of the whole hot path (Algorithm 2, PAPER.md:152-156:
sample the batches, gather, Gram, m greedy select/deflate steps per batch,
union, merge TED) over the synthetic AutoTVM conv2d pool of the config.
Weak scaling: every rank runs cfg.B batches of M points per step
(B_total = N_gpus * cfg.B), then the winners are all-gathered and merged.
value = batch selections per second, whole job = steps * B_total * m / time
(the merge TED's selections are NOT counted; its time is).

Timing: W >= 3 untimed warm-up steps; barrier + cuda synchronize; CUDA events
on the library's stream around exactly K steps; max over ranks.  Inputs are
larger than L2 (K = 4 M^2 bytes = 1 GiB per batch at M = 16384, vs 126 MB L2).
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import tempfile
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

METRIC = "BTED selected points/sec and deflate-step HBM GB/s vs roofline at 1/2/4/8 B200"
UNIT = "points/s"
K2_NAME = {"dense": "deflate_rescore_kernel",
           "packed": "deflate_packed_ldg_kernel (+ finalize_packed_kernel, per step)",
           "implicit": "tile_pass_kernel (q = K l on the read-only packed K; per step incl. ell_kernel + fin64_kernel)"}
LAYOUT_FLAG = {"dense": 4, "packed": 64, "implicit": 0}          # BTED_FLAG_DENSE / _LITERAL / default
ALG_BYTES_PER_N2 = {"dense": 8.0, "packed": 4.0, "implicit": 2.0}


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--config", default="resnet18")
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--cpu-budget-s", type=float, default=15.0)
    ap.add_argument("--scaling", default="weak", choices=["weak", "strong"],
                    help="weak: every GPU runs the config's B batches; strong: the config's B batches are split")
    ap.add_argument("--shard-engine", default="implicit", choices=["implicit", "dense"],
                    help="oversized config on N > 1 GPUs (or with --sharded): the tile-sharded implicit engine "
                         "(one q all-reduce per step, ~2 N^2 / P B per GPU) or the dense row bands "
                         "(key all-reduce + pivot all-gather per step, 8 N^2 / P B per GPU)")
    ap.add_argument("--sharded", action="store_true",
                    help="run the oversized config through the multi-GPU sharded driver even at one GPU")
    ap.add_argument("--norm-mode", default="symmetric", choices=["symmetric", "literal"],
                    help="oversized row-sharded mode: scores from the band's row norms (default) or the "
                         "north_star's literal all-reduce(SUM) of partial column norms")
    ap.add_argument("--persistent", action="store_true",
                    help="implicit engine: run the m-1 steps as one persistent kernel (BTED_FLAG_PERSISTENT_LOOP)")
    ap.add_argument("--layout", default="implicit", choices=["packed", "dense", "implicit"],
                    help="engine: implicit deflation on the read-only packed K (2 N^2 B/step, the default), "
                         "literal deflation on packed upper-triangular tiles (4 N^2 B/step) or dense (8 N^2 B/step)")
    return ap.parse_args()


def peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        with open(p) as f:
            j = json.load(f)
        return float(j["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs: torch copy, read+write bytes)"
    return 6650.0, "fallback (B200_PROFILING.md: 6.65 TB/s)"


# ------------------------------------------------------------------ clocks
class Clocks:
    FIELDS = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
              "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
              "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, index: int):
        self.index = index
        self.f = tempfile.NamedTemporaryFile("w+", suffix=".csv", delete=False)
        self.p = None

    def start(self):
        try:
            self.p = subprocess.Popen(["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.FIELDS}",
                                       "--format=csv,noheader,nounits", "-lms", "200"],
                                      stdout=self.f, stderr=subprocess.DEVNULL)
        except Exception:
            self.p = None
        time.sleep(0.3)

    def stop(self):
        if self.p is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        time.sleep(0.25)
        self.p.terminate()
        try:
            self.p.wait(timeout=5)
        except Exception:
            self.p.kill()
        self.f.flush()
        self.f.seek(0)
        sm, smax, reasons = [], [], set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for line in self.f.read().splitlines():
            c = [x.strip() for x in line.split(",")]
            if len(c) < 9:
                continue
            try:
                sm.append(float(c[1]))
                smax.append(float(c[2]))
            except ValueError:
                continue
            for n, v in zip(names, c[5:9]):
                if v.lower().startswith("active"):
                    reasons.add(n)
        os.unlink(self.f.name)
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(smax) if smax else None,
                "reasons": sorted(reasons), "samples": len(sm)}


# ------------------------------------------------------------------ CPU oracle timing
def oracle_points_per_s(Xb: np.ndarray, gamma: float, mu: float, m: int, budget_s: float):
    """The fp64 oracle (oracle/ted_dense.c, all host cores) on one full batch:
    Gram + as many of the m greedy steps as fit in ~budget_s; the m-step TED
    time is extrapolated from the measured per-step time.  Batches above
    32768 points use the matrix-free O2 oracle (oracle/ted_matfree.c): a 1-step
    and a 3-step run, the per-step time from their difference."""
    if Xb.shape[0] > 32768:
        from oracle import matfree
        t0 = time.perf_counter()
        matfree.ted(Xb, gamma, mu, 1)
        t1 = time.perf_counter() - t0
        t0 = time.perf_counter()
        matfree.ted(Xb, gamma, mu, 3)
        t3 = time.perf_counter() - t0
        per = max((t3 - t1) / 2, 1e-9)
        t_ted = t1 + (m - 1) * per
        return m / t_ted, t1, per, 3, matfree.num_threads()
    from oracle import dense
    t0 = time.perf_counter()
    K = dense.gram(Xb, gamma)
    t_gram = time.perf_counter() - t0
    steps, t_steps = 0, 0.0
    while steps < m and (steps == 0 or t_steps < budget_s):
        t1 = time.perf_counter()
        # one greedy step of Alg. 1 on the current (in-place deflated) K
        dense.ted_on_matrix(K, mu, 1)
        t_steps += time.perf_counter() - t1
        steps += 1
    del K
    t_ted = t_gram + m * (t_steps / steps)
    return m / t_ted, t_gram, t_steps / steps, steps, dense.num_threads()


def bench_reference(args):
    """--impl reference: the oracle IS the reference arm (no reference code exists)."""
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    from oracle.sampling import sample_batches
    from synth import config_pool
    X, gamma, cfg = config_pool(args.config)
    mu = float(np.float32(cfg["mu"]))
    V = sample_batches(X.shape[0], cfg["M"], 1, cfg["seed"])[0]
    Xb = X[V]
    budget = max(1.0, min(args.cpu_budget_s, 10.0))
    vals, times = [], []
    for it in range(args.warmup + args.steps):
        t0 = time.perf_counter()
        v, tg, ts, n, cores = oracle_points_per_s(Xb, gamma, mu, cfg["m"], budget_s=budget / 4)
        if it >= args.warmup:
            vals.append(v)
            times.append(time.perf_counter() - t0)
    value = float(statistics.median(vals))
    sample = (f"per step: oracle Gram of batch 0 (N={cfg['M']}, d={cfg['d']}) + {n} of {cfg['m']} greedy "
              f"steps; points/s extrapolated to the full {cfg['m']}-step TED (batch selections only)")
    line = {"impl": "reference", "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * float(np.mean(times)),
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f64",
            "data": "synthetic", "config": workload_config(args.config, cfg, gamma, 1),
            "cpu_baseline": {"value": value, "unit": UNIT, "cores": cores, "kind": "oracle", "sample": sample},
            "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


L2_BYTES = 126 << 20          # B200 L2 (126 MB)


def workload_config(name, cfg, gamma, world, B=None):
    B = cfg["B"] * world if B is None else B
    return {"workload": f"{name}: BTED on the AutoTVM conv2d knob pool of {cfg['workload']} "
                        f"(P={cfg['pool']} configs, d={cfg['d']}), B={B} batches of "
                        f"M={cfg['M']}, m={cfg['m']}, mu={cfg['mu']}, RBF gamma={gamma:.6g} (median heuristic)",
            "pool": cfg["pool"], "M": cfg["M"], "d": cfg["d"], "m": cfg["m"], "B": B,
            "batches_per_gpu": B / world, "mu": cfg["mu"], "seed": cfg["seed"],
            "l2": f"inputs larger than L2: K = 4*M^2 = {4 * cfg['M'] ** 2} bytes per batch > {L2_BYTES >> 20} MiB",
            "parallelism": f"batch round-robin over {world} GPU(s)" if world > 1 else "1 GPU"}


# ------------------------------------------------------------------ ours
def bench_ours(args):
    import torch
    import paper_conf_date_sunbg021_b200 as bt
    from paper_conf_date_sunbg021_b200 import _lib as L
    from paper_conf_date_sunbg021_b200.dist import TorchComm, run_batches_dp
    from synth import config_pool

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    comm = None
    if world > 1 or args.sharded:
        import torch.distributed as dist
        if world == 1:                                   # --sharded on one GPU: a one-rank NCCL group
            import socket
            sk = socket.socket()
            sk.bind(("127.0.0.1", 0))
            os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
            os.environ.setdefault("MASTER_PORT", str(sk.getsockname()[1]))
            sk.close()
            os.environ.setdefault("RANK", "0")
            os.environ.setdefault("WORLD_SIZE", "1")
        # a dead or stalled rank fails the job instead of hanging it: NCCL async error
        # handling + a collective timeout (BTED_NCCL_TIMEOUT_S, default 600 s)
        os.environ.setdefault("TORCH_NCCL_ASYNC_ERROR_HANDLING", "1")
        import datetime
        dist.init_process_group("nccl", device_id=dev, timeout=datetime.timedelta(
            seconds=float(os.environ.get("BTED_NCCL_TIMEOUT_S", "600"))))
        comm = TorchComm()

    if args.config == "wholemodel":
        return bench_wholemodel(args, comm, dev, world, rank, local)
    X, gamma, cfg = config_pool(args.config)
    mu = float(np.float32(cfg["mu"]))
    M, m, d, P = cfg["M"], cfg["m"], cfg["d"], X.shape[0]
    if cfg["B"] == 1 and args.config == "oversized" and (world > 1 or args.sharded):
        return bench_sharded(args, X, gamma, cfg, comm, dev, world, rank)
    B = cfg["B"] * world if args.scaling == "weak" else cfg["B"]
    stream = torch.cuda.Stream(dev)
    X_dev = torch.from_numpy(X).to(dev)
    torch.cuda.synchronize()
    lay_flag = LAYOUT_FLAG[args.layout] | (256 if args.persistent else 0)
    pool = bt.CandidateSet(X_dev, gamma, num_batches=B, seed=cfg["seed"], device=local,
                           flags=L.BTED_FLAG_TIMING | lay_flag, stream=stream.cuda_stream)

    def step():
        if world == 1:
            return pool.run_batches(M, m, mu, want_batches=False)[0]
        with torch.cuda.stream(stream):
            return run_batches_dp(pool.ctx, M, m, mu, B, comm, dev)[0]

    def barrier():
        if world > 1:
            torch.distributed.barrier()

    def max_over_ranks(v: float) -> float:
        if world == 1:
            return v
        t = torch.tensor([v], dtype=torch.float64, device=dev)
        torch.distributed.all_reduce(t, op=torch.distributed.ReduceOp.MAX)
        return float(t.item())

    l2_flush = 4 * cfg["M"] ** 2 < L2_BYTES
    if l2_flush:
        flush_buf = torch.empty(2 * L2_BYTES, dtype=torch.uint8, device=dev)
        l2_note = (f"K = 4*M^2 = {4 * cfg['M'] ** 2} bytes per batch fits in L2: a {2 * L2_BYTES >> 20} MiB "
                      f"buffer is written before every timed step (outside its CUDA events)")
    for _ in range(args.warmup):
        step()
    L.bted_reset_stats(pool.ctx)
    clocks = Clocks(local)
    clocks.start()
    l0 = bt.bted_kernel_launches()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    barrier()
    torch.cuda.synchronize()
    if l2_flush:
        # K (4 M^2 bytes per batch) fits in L2: write a buffer larger than L2
        # before every step, outside the per-step events, and sum the steps
        ms_sum = 0.0
        for _ in range(args.steps):
            with torch.cuda.stream(stream):
                flush_buf.fill_(1)
            e0.record(stream)
            sel = step()
            e1.record(stream)
            torch.cuda.synchronize()
            ms_sum += e0.elapsed_time(e1)
    else:
        e0.record(stream)
        for _ in range(args.steps):
            sel = step()
        e1.record(stream)
        torch.cuda.synchronize()
    barrier()
    launches = bt.bted_kernel_launches() - l0
    ms = max_over_ranks(ms_sum if l2_flush else e0.elapsed_time(e1))
    clk = clocks.stop()
    stats = L.bted_get_stats(pool.ctx)
    value = args.steps * B * m / (ms / 1e3)

    # roofline of the dominant kernel K2 (fused deflate + rescore), live events
    peak, peak_src = peaks()
    traffic = None
    if stats["k2_launches"] > 0:
        k2_avg_ms = stats["k2_ms"] / stats["k2_launches"]
        # algorithmic bytes per step: fp32 read + write of K = 8 N^2 (dense) or of
        # its upper triangle = 4 N^2 (packed; report against 4 N^2)
        alg_bytes = ALG_BYTES_PER_N2[args.layout] * M * M
        achieved = alg_bytes / (k2_avg_ms / 1e3) / 1e9
        tj = os.path.join(ROOT, "profiles", "k2_traffic.json")
        if os.path.exists(tj):
            with open(tj) as f:
                tjd = json.load(f)
            ent = tjd.get(args.layout, {})
            if ent.get("M") == M:
                traffic = ent.get("dram_bytes_per_launch")
        roofline = {"bound": "hbm", "kernel": K2_NAME[args.layout], "achieved": achieved, "peak": peak,
                    "unit": "GB/s", "frac": achieved / peak, "traffic": traffic,
                    "frac_of_8TBs": achieved / 8000.0, "peak_source": peak_src,
                    "alg_bytes_per_launch": alg_bytes, "avg_launch_ms": k2_avg_ms,
                    "launches_timed": stats["k2_launches"],
                    "k2_share_of_step": (stats["k2_ms"] / ms) if ms > 0 else None,
                    "k1_ms_per_batch": stats["k1_ms"] / max(stats["teds"], 1)}
    else:
        # small batches: every TED is one cluster kernel with K in distributed
        # shared memory -- no HBM stream to hold against the HBM roofline
        roofline = {"bound": "latency", "kernel": "ted_cluster_kernel (K in DSMEM, whole TED per launch)",
                    "achieved": None, "peak": None, "unit": None, "frac": None, "traffic": None,
                    "small_teds_timed": stats["small_teds"],
                    "ms_per_small_launch": stats["small_ms"] / max(args.steps, 1),
                    "small_share_of_step": (stats["small_ms"] / ms) if ms > 0 else None}

    # end to end through the public API with HOST buffers (pinned), per step:
    # H2D of that step's pool, the whole BTED, D2H of the result.  Two contexts
    # on two streams alternate, so the copy of step k+1's pool overlaps step k's
    # compute (how a tuner streaming node pools would drive the API).  Timed
    # with the host wall clock around exactly K steps (every copy included).
    e2e = None
    if not args.no_e2e:
        import time as _time
        pins, ctxs2, strs = [], [], []
        for q in range(2):
            pa = L.PinnedArray(X.shape)          # page-locked memory of the library's runtime
            pa.array[:] = X
            sq = torch.cuda.Stream(dev)
            pins.append(pa)
            strs.append(sq)
            ctxs2.append(bt.CandidateSet(pa.array, gamma, num_batches=B, seed=cfg["seed"], device=local,
                                         flags=lay_flag, stream=sq.cuda_stream))

        def e2e_step(k, K):
            cur = ctxs2[k % 2]
            if k + 1 < K:
                L.bted_update(ctxs2[(k + 1) % 2].ctx, pins[(k + 1) % 2].ptr)   # async H2D, next pool
            if world == 1:
                return cur.run_batches(M, m, mu, want_batches=False)[0]       # ends with the D2H
            with torch.cuda.stream(strs[k % 2]):
                return run_batches_dp(cur.ctx, M, m, mu, B, comm, dev)[0]

        for k in range(max(1, args.warmup)):
            if k == 0:
                L.bted_update(ctxs2[0].ctx, pins[0].ptr)
            e2e_step(k, max(1, args.warmup))
        barrier()
        torch.cuda.synchronize()
        t0 = _time.perf_counter()
        L.bted_update(ctxs2[0].ctx, pins[0].ptr)
        for k in range(args.steps):
            e2e_step(k, args.steps)
        torch.cuda.synchronize()
        barrier()
        ems = max_over_ranks((_time.perf_counter() - t0) * 1e3)
        for c in ctxs2:
            c.close()
        for pa in pins:
            pa.close()
        e2e = {"value": args.steps * B * m / (ems / 1e3), "unit": UNIT,
               "h2d_bytes_per_step": int(P * d * 4),
               "d2h_bytes_per_step": int(8 * m + 4 + 8 * m + 4 + 4),
               "timer": "host wall clock; step k+1's pool H2D overlaps step k on a second stream"}

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        from oracle.sampling import sample_batches
        V = sample_batches(P, M, 1, cfg["seed"])[0]
        v, tg, ts, n, cores = oracle_points_per_s(X[V], gamma, mu, m, args.cpu_budget_s)
        which = "matrix-free O2 C/OpenMP oracle" if M > 32768 else "dense C/OpenMP oracle"
        cpu = {"value": v, "unit": UNIT, "cores": cores, "kind": "oracle",
               "sample": (f"batch 0 (N={M}): fp64 Gram ({tg:.2f} s) + {n} of {m} greedy steps "
                          f"({ts:.3f} s/step) with the {which}; points/s of the full "
                          f"{m}-step TED extrapolated from those")}

    pool.close()
    if rank == 0:
        line = {"metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
                "warmup": args.warmup, "ms_per_step": ms / args.steps, "higher_is_better": True,
                "scaling": args.scaling, "vs_baseline": None, "dtype": "f32", "data": "synthetic",
                "config": dict(workload_config(args.config, cfg, gamma, world, B),
                               **({"l2": l2_note} if l2_flush else {})),
                "layout": args.layout,
                "roofline": roofline,
                "cpu_baseline": cpu, "e2e": e2e, "gpu_launches": int(launches), "clocks": clk,
                "final_selection_head": [int(x) for x in sel[:8]]}
        print(json.dumps(line), flush=True)
    if world > 1:
        torch.distributed.destroy_process_group()


def bench_wholemodel(args, comm, dev, world, rank, local):
    """config 'wholemodel': ResNet-50 + MobileNet-v2, 40 tunable nodes (each its
    own knob-space pool), BTED with B = 4 batches of M = 32768, m = 64 per node.
    Nodes go round-robin over the ranks (independent BTEDs: no data-path
    collective); a step = every node's BTED once.  Strong scaling (fixed work)."""
    import torch
    import paper_conf_date_sunbg021_b200 as bt
    from paper_conf_date_sunbg021_b200 import _lib as L
    from synth import CONFIGS, MU, whole_model_nodes, whole_model_pools
    cfg = dict(CONFIGS["wholemodel"])
    mu = float(np.float32(MU))
    M, m, B = cfg["M"], cfg["m"], cfg["B"]
    nodes = whole_model_nodes()
    mine = [k for k in range(len(nodes)) if k % world == rank]
    pools = whole_model_pools(which=mine)
    stream = torch.cuda.Stream(dev)
    ctxs = []
    for (wl, X, g), k in zip(pools, mine):
        Xd = torch.from_numpy(X).to(dev)
        ctxs.append((bt.CandidateSet(Xd, g, num_batches=B, seed=cfg["seed"] + k, device=local,
                                     flags=L.BTED_FLAG_TIMING | LAYOUT_FLAG[args.layout],
                                     stream=stream.cuda_stream), Xd))
    torch.cuda.synchronize()

    def step():
        for cs, _ in ctxs:
            cs.run_batches(min(M, cs.N), m, mu, want_batches=False)

    for _ in range(args.warmup):
        step()
    for cs, _ in ctxs:
        L.bted_reset_stats(cs.ctx)
    clocks = Clocks(local)
    clocks.start()
    l0 = bt.bted_kernel_launches()
    if world > 1:
        torch.distributed.barrier()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(stream)
    for _ in range(args.steps):
        step()
    e1.record(stream)
    torch.cuda.synchronize()
    if world > 1:
        torch.distributed.barrier()
    launches = bt.bted_kernel_launches() - l0
    ms = e0.elapsed_time(e1)
    if world > 1:
        t = torch.tensor([ms], dtype=torch.float64, device=dev)
        torch.distributed.all_reduce(t, op=torch.distributed.ReduceOp.MAX)
        ms = float(t.item())
    clk = clocks.stop()
    k2_ms = k2_n = 0
    for cs, _ in ctxs:
        stt = L.bted_get_stats(cs.ctx)
        k2_ms += stt["k2_ms"]
        k2_n += stt["k2_launches"]
    peak, peak_src = peaks()
    k2_avg = k2_ms / max(k2_n, 1)
    alg = ALG_BYTES_PER_N2[args.layout] * M * M
    total_sel = args.steps * len(nodes) * B * m
    for cs, _ in ctxs:
        cs.close()
    if rank == 0:
        line = {"metric": METRIC, "value": total_sel / (ms / 1e3), "unit": UNIT, "n_gpus": world,
                "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms / args.steps,
                "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "f32",
                "data": "synthetic", "layout": args.layout,
                "config": {"workload": f"wholemodel: ResNet-50 + MobileNet-v2, {len(nodes)} conv nodes (own knob "
                                       f"pools, P = min(2^20, |D|)), B={B} x M={M}, m={m} per node",
                           "nodes": len(nodes), "B_per_node": B, "M": M, "m": m, "mu": MU,
                           "l2": "inputs larger than L2 (K = 4 M^2 bytes per batch)",
                           "parallelism": f"nodes round-robin over {world} GPU(s)"},
                "roofline": {"bound": "hbm", "kernel": K2_NAME[args.layout], "achieved": alg / (k2_avg / 1e3) / 1e9,
                             "peak": peak, "unit": "GB/s", "frac": alg / (k2_avg / 1e3) / 1e9 / peak,
                             "traffic": None, "peak_source": peak_src, "alg_bytes_per_launch": alg,
                             "avg_launch_ms": k2_avg, "launches_timed": k2_n},
                "cpu_baseline": None, "e2e": None, "gpu_launches": int(launches), "clocks": clk}
        print(json.dumps(line), flush=True)
    if world > 1:
        torch.distributed.destroy_process_group()


def bench_sharded(args, X, gamma, cfg, comm, dev, world, rank):
    """config 'oversized' on N > 1 GPUs: ONE batch of M points over the ranks.
    Default (--shard-engine implicit): the packed Gram tiles split k mod P, one
    all-reduce(SUM) of q = K l per step -- dist.ShardedImplicitTed.  With
    --shard-engine dense: K row-sharded in bands, per step an 8-byte MAX
    all-reduce of the packed argmax key and an all-gather of column s (= row s)
    -- dist.ShardedTed (--norm-mode literal adds the column-norm all-reduce)."""
    import torch
    import paper_conf_date_sunbg021_b200 as bt
    from paper_conf_date_sunbg021_b200.dist import LibShard, ShardedTed, band
    mu = float(np.float32(cfg["mu"]))
    M, m = cfg["M"], cfg["m"]
    # the batch V_0 = the first draw of Alg. 2 l.2, gathered on every rank by the library
    V = bt.bted_sample_batches(X.shape[0], M, 1, cfg["seed"])[0]
    Xb = np.ascontiguousarray(X[V])
    stream = torch.cuda.Stream(dev)
    implicit = args.shard_engine == "implicit"
    if implicit:
        from paper_conf_date_sunbg021_b200.dist import LibIShard, ShardedImplicitTed
        shard = LibIShard(Xb, M, cfg["d"], gamma, rank, world, dev, stream)
        st = ShardedImplicitTed(shard, M, comm, dev, stream, graph=True)
    else:
        r0, r1, _ = band(M, world, rank)
        shard = LibShard(Xb, M, cfg["d"], gamma, r0, r1, dev, stream)
        st = ShardedTed(shard, M, comm, dev, stream, graph=True, norm_mode=args.norm_mode)
    lw = bt.bted_kernel_launches()
    st.select(m, mu)                                     # first call: one eager loop + the graph capture
    per_select = (bt.bted_kernel_launches() - lw) // 2   # (graph replays do not pass the launch counter)
    for _ in range(args.warmup - 1):
        st.select(m, mu)
    clocks = Clocks(int(os.environ.get("LOCAL_RANK", "0")))
    clocks.start()
    l0 = bt.bted_kernel_launches()
    torch.distributed.barrier()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(stream)
    for _ in range(args.steps):
        idx, _ = st.select(m, mu)
    e1.record(stream)
    torch.cuda.synchronize()
    torch.distributed.barrier()
    launches = bt.bted_kernel_launches() - l0 + per_select * args.steps
    t = torch.tensor([e0.elapsed_time(e1)], dtype=torch.float64, device=dev)
    torch.distributed.all_reduce(t, op=torch.distributed.ReduceOp.MAX)
    ms = float(t.item())
    clk = clocks.stop()
    shard.close()
    peak, peak_src = peaks()
    step_ms = ms / args.steps / max(m - 1, 1)
    per_gpu_bytes = (2.0 if implicit else 8.0) * M * M / world
    achieved = per_gpu_bytes / (step_ms / 1e3) / 1e9
    if rank == 0:
        line = {"metric": METRIC, "value": args.steps * m / (ms / 1e3), "unit": UNIT, "n_gpus": world,
                "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms / args.steps,
                "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "f32",
                "data": "synthetic", "layout": "implicit-tile-sharded" if implicit else "dense-row-sharded",
                "config": dict(workload_config(args.config, cfg, gamma, world, 1),
                               norm_mode=None if implicit else args.norm_mode,
                               parallelism=(f"Gram tiles k = rank mod {world} over {world} GPUs (one NCCL all-reduce "
                                            "of q = K l per step)") if implicit else
                               f"row-sharded K over {world} GPUs (NCCL all-reduce + all-gather per step)"),
                "roofline": {"bound": "hbm",
                             "kernel": ("tile_pass_kernel (own tiles) + ell + fin64 + NCCL" if implicit else
                                        "deflate_rescore_kernel (per-GPU band) + NCCL"),
                             "achieved": achieved, "peak": peak, "unit": "GB/s", "frac": achieved / peak,
                             "traffic": None, "peak_source": peak_src,
                             "alg_bytes_per_launch": per_gpu_bytes, "avg_launch_ms": step_ms,
                             "note": ("per-GPU step time (Gram + head amortised) includes the q all-reduce"
                                      if implicit else "per-GPU step time includes the two collectives")},
                "cpu_baseline": None, "e2e": None, "gpu_launches": int(launches), "clocks": clk,
                "final_selection_head": [int(x) for x in idx[:8]]}
        print(json.dumps(line), flush=True)
    torch.distributed.destroy_process_group()


def spawn_ranks(n: int) -> int:
    """`python bench.py --gpus N` outside torchrun: re-launch this command as N
    ranks (one process per GPU) under torch.distributed.run on 127.0.0.1."""
    import socket
    sk = socket.socket()
    sk.bind(("127.0.0.1", 0))
    port = sk.getsockname()[1]
    sk.close()
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={n}",
           "--master-addr=127.0.0.1", f"--master-port={port}", os.path.abspath(__file__), *sys.argv[1:]]
    return subprocess.call(cmd)


def main():
    args = parse()
    if args.warmup < 3:
        print("warning: --warmup < 3 violates the timing rules; using 3", file=sys.stderr)
        args.warmup = 3
    if args.gpus > 1 and "WORLD_SIZE" not in os.environ:
        sys.exit(spawn_ranks(args.gpus))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    if world != args.gpus:
        sys.exit(f"bench.py: --gpus {args.gpus} but WORLD_SIZE={world} (launch one rank per GPU)")
    if args.impl == "reference":
        bench_reference(args)
    else:
        bench_ours(args)


if __name__ == "__main__":
    main()
