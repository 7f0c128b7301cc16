#!/usr/bin/env python
"""Benchmark of the B200 CART hot path (BASELINE.json metric: tree-fit row.feature split
evals/s and DSE predictions/s).

Workload (N=1): BASELINE.json configs[1] -- 1M rows x 16 features (schema S16, seed 1),
max_depth 12, min_samples_leaf 1; one step = dt_fit on the training table + fused
dt_predict_eval on a 1M-row held-out table (seed 2).  value = split evals / step time
(split evals = sum over searched nodes of N*d).  Inputs are resident in HBM; L2 is
flushed (256 MB write) between timed steps, outside the per-step CUDA events.
N>1 (torchrun, or --gpus N, which re-launches itself through torch.distributed.run): the
headline is BASELINE configs[2] -- ONE 100M x 32 (S32, seed 3), depth-16 fit row-sharded
over the N ranks (dt_fit_sharded over NCCL: value-range presort, per-level allgathers of
node bests and boundary records, OR-allreduce of the go-left bitmap), strong scaling,
device-timed, max over ranks; independent configs[1] replicas are an extra key.

Also reported: e2e (same metric through the C-ABI with host buffers, H2D/D2H inside the
timed region), DSE predictions/s (BASELINE configs[3] shape on one GPU: 2^28 materialised
candidates by default, depth-20 / min_samples_leaf-128 tree; and the full 2^30 cross
product through the factored predictor), the dominant kernel's roofline, the oracle timed
on the host as cpu_baseline, configs[0] LOO, configs[4] grid, configs[2] (100M x 32,
depth 16) on one GPU (row-sharded over NCCL at N>1: the N>1 headline), a 16-tree Random Forest and
KNN regression.

--impl reference: the oracle (the slow CPU reference of this tier) timed on the host.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "tree-fit row·feature split evals/s and DSE predictions/s at 1/2/4/8 B200"
N_TRAIN = 1_000_000
D = 16
MAX_DEPTH = 12
MIN_LEAF = 1
CPU_SAMPLE_ROWS = 250_000
REF_SAMPLE_ROWS = 100_000
FALLBACK_HBM_GBS = 6650.0

REASONS = {0x1: "gpu_idle", 0x2: "applications_clocks_setting", 0x4: "sw_power_cap",
           0x8: "hw_slowdown", 0x10: "sync_boost", 0x20: "sw_thermal_slowdown",
           0x40: "hw_thermal_slowdown", 0x80: "hw_power_brake_slowdown",
           0x100: "display_clocks_setting"}


def parse():
    p = argparse.ArgumentParser()
    p.add_argument("--gpus", type=int, default=1)
    p.add_argument("--steps", type=int, default=50)
    p.add_argument("--warmup", type=int, default=5)
    p.add_argument("--impl", default="ours", choices=["ours", "reference"])
    p.add_argument("--dse-log2", type=int, default=28, help="log2 of DSE candidates (30 = full C4)")
    p.add_argument("--no-dse", action="store_true")
    p.add_argument("--no-cpu", action="store_true")
    p.add_argument("--e2e-steps", type=int, default=30,
                   help="e2e steps (double-buffered: the first upload is a pipeline fill inside the region)")
    p.add_argument("--no-extra", action="store_true", help="skip configs[0] LOO and configs[4] grid")
    p.add_argument("--grid-rows", type=int, default=10_000_000, help="configs[4] rows (0 = skip)")
    p.add_argument("--c3-rows", type=int, default=100_000_000,
                   help="configs[2] rows (x 32 features, depth 16; 0 = skip)")
    p.add_argument("--force-sharded", action="store_true",
                   help="run the N>1 headline (row-sharded configs[2] over NCCL) even with one rank")
    p.add_argument("--sharded-local", type=int, default=0,
                   help="N=1 only: also time a row-sharded fit with this many thread ranks on the GPU")
    return p.parse_args()


def workload_config(world):
    return {"workload": "configs[1]: 1M x 16 (S16 CNN x GPU table, seed 1), max_depth 12, "
                        "min_samples_leaf 1; step = dt_fit + dt_predict_eval on 1M held-out rows",
            "n_train": N_TRAIN, "n_eval": N_TRAIN, "d": D, "max_depth": MAX_DEPTH,
            "min_samples_leaf": MIN_LEAF, "l2": "flushed (256 MB write) between timed steps",
            "parallelism": "replicas" if world > 1 else "single", "ranks": world}


def peaks():
    path = os.path.join(ROOT, "MEASURED_PEAKS.json")
    try:
        with open(path) as fh:
            return float(json.load(fh)["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    except Exception:
        return FALLBACK_HBM_GBS, "fallback (B200_PROFILING.md)"


class ClockSampler:
    """NVML sampling of SM clock and clock-event reasons during the timed region."""

    def __init__(self, index=0, period=0.01):
        self.index, self.period = index, period
        self.samples, self.reasons = [], 0
        self.max_mhz = None
        self._stop = threading.Event()
        self._t = None

    def __enter__(self):
        try:
            import pynvml
            pynvml.nvmlInit()
            h = pynvml.nvmlDeviceGetHandleByIndex(self.index)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(h, pynvml.NVML_CLOCK_SM)

            def run():
                while not self._stop.is_set():
                    try:
                        self.samples.append(pynvml.nvmlDeviceGetClockInfo(h, pynvml.NVML_CLOCK_SM))
                        self.reasons |= int(pynvml.nvmlDeviceGetCurrentClocksEventReasons(h))
                    except Exception:
                        pass
                    time.sleep(self.period)

            self._t = threading.Thread(target=run, daemon=True)
            self._t.start()
        except Exception:
            self._t = None
        return self

    def __exit__(self, *a):
        self._stop.set()
        if self._t:
            self._t.join()

    def summary(self):
        names = [v for k, v in REASONS.items() if self.reasons & k and v != "gpu_idle"]
        return {"sm_mhz": statistics.median(self.samples) if self.samples else None,
                "sm_max_mhz": self.max_mhz, "reasons": names, "samples": len(self.samples)}


def dist_init():
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if world > 1:
        import torch
        import torch.distributed as dist
        torch.cuda.set_device(local)
        dist.init_process_group("nccl")
    elif "--force-sharded" in sys.argv:  # one-rank process group for the NCCL id broadcast
        import torch.distributed as dist
        os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
        os.environ.setdefault("MASTER_PORT", "29511")
        dist.init_process_group("gloo", rank=0, world_size=1)
    return world, rank, local


def max_over_ranks(x, world):
    if world == 1:
        return x
    import torch
    import torch.distributed as dist
    t = torch.tensor([x], dtype=torch.float64, device="cuda")
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


def sum_over_ranks(x, world):
    if world == 1:
        return x
    import torch
    import torch.distributed as dist
    t = torch.tensor([x], dtype=torch.float64, device="cuda")
    dist.all_reduce(t, op=dist.ReduceOp.SUM)
    return float(t.item())


def barrier(world):
    if world > 1:
        import torch.distributed as dist
        dist.barrier()


# ---------------------------------------------------------------------- oracle (CPU) --

def _one_core():
    """Pin this process to one host core for a CPU timing; returns the previous mask."""
    try:
        prev = os.sched_getaffinity(0)
        os.sched_setaffinity(0, {min(prev)})
        return prev
    except (AttributeError, OSError):
        return None


def _cpu_model():
    try:
        with open("/proc/cpuinfo") as fh:
            for line in fh:
                if line.startswith("model name"):
                    return line.split(":", 1)[1].strip()
    except OSError:
        pass
    return "unknown"


def oracle_rate(rows: int, seed: int = 1):
    """Oracle fit on the first `rows` rows of the workload table, pinned to one host core;
    returns (evals/s, s, evals, sklearn) where sklearn is DecisionTreeRegressor's time on
    the same sample (the paper's presumed tool) or None."""
    import datagen
    import oracle
    X, y = datagen.cnn_gpu_table(seed, rows)
    prev = _one_core()
    try:
        t0 = time.perf_counter()
        _, ev = oracle.fit(X, y, MAX_DEPTH, MIN_LEAF, return_evals=True)
        dt = time.perf_counter() - t0
        sk = None
        try:
            from sklearn.tree import DecisionTreeRegressor
            t1 = time.perf_counter()
            DecisionTreeRegressor(max_depth=MAX_DEPTH, min_samples_leaf=MIN_LEAF).fit(X, y)
            ts = time.perf_counter() - t1
            sk = {"value": ev / ts, "unit": "split evals/s", "seconds": ts,
                  "note": "sklearn DecisionTreeRegressor (Cython, single thread), same sample and numerator"}
        except ImportError:
            pass
    finally:
        if prev:
            os.sched_setaffinity(0, prev)
    return ev / dt, dt, ev, sk


def run_reference(args, world, rank):
    if rank != 0:
        return
    import datagen
    import oracle
    oracle.build()
    X, y = datagen.cnn_gpu_table(1, REF_SAMPLE_ROWS)
    prev = _one_core()
    for _ in range(args.warmup):
        oracle.fit(X, y, MAX_DEPTH, MIN_LEAF)
    t0 = time.perf_counter()
    ev_tot = 0
    for _ in range(args.steps):
        _, ev = oracle.fit(X, y, MAX_DEPTH, MIN_LEAF, return_evals=True)
        ev_tot += ev
    dt = time.perf_counter() - t0
    if prev:
        os.sched_setaffinity(0, prev)
    v = ev_tot / dt
    sample = (f"oracle fit (single-threaded C, -O2) on the first {REF_SAMPLE_ROWS} rows of the "
              f"configs[1] table (seed 1), depth {MAX_DEPTH}; per step")
    line = {"impl": "reference", "metric": METRIC, "value": v, "unit": "split evals/s",
            "n_gpus": world, "steps": args.steps, "warmup": args.warmup,
            "ms_per_step": dt / args.steps * 1e3, "higher_is_better": True, "scaling": "weak",
            "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": dict(workload_config(1), n_train=REF_SAMPLE_ROWS,
                           sample=f"bounded sample: each step fits the first {REF_SAMPLE_ROWS} of the "
                                  f"{N_TRAIN} configs[1] rows (a 1M-row oracle fit takes ~20 s)"),
            "cpu_baseline": {"value": v, "unit": "split evals/s", "cores": 1, "kind": "oracle",
                             "sample": sample, "cpu_model": _cpu_model(),
                             "host_cores_available": os.cpu_count()},
            "e2e": {"value": v, "unit": "split evals/s", "h2d_bytes_per_step": 0,
                    "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


# ---------------------------------------------------------------------- ours (GPU) ----

def sharded_fit_measure(args, rank, dev, X, y, stream):
    """--sharded-local P (N=1): the configs[1] table row-sharded over P host-thread ranks
    sharing this GPU (dt_comm_init_local): a functional check of the sharded path, timed
    by the host clock (the ranks share one GPU, so this is no scaling number)."""
    import threading

    import torch

    import paper_conf_ipps_metzgd23_b200 as dt
    P = args.sharded_local
    comms = dt.dt_comm_init_local(P)
    n = X.shape[0]
    cuts = [(r * n) // P for r in range(P + 1)]
    steps = max(3, min(args.steps, 10))

    def one_round():
        trees = [None] * P

        def run(i):
            s = torch.cuda.Stream()
            with torch.cuda.stream(s):
                a, b = cuts[i], cuts[i + 1]
                trees[i] = dt.dt_fit_sharded(comms[i], X[a:b], y[a:b], a, n, MAX_DEPTH, MIN_LEAF, stream=s)
        th = [threading.Thread(target=run, args=(i,)) for i in range(P)]
        for t in th:
            t.start()
        for t in th:
            t.join()
        return trees

    one_round()
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    for _ in range(steps):
        trees = one_round()
    torch.cuda.synchronize()
    dt_s = time.perf_counter() - t0
    ref = dt.dt_fit(X, y, MAX_DEPTH, MIN_LEAF).nodes
    same = all(np.array_equal(t.nodes[k], ref[k]) for t in trees
               for k in ("feature", "left", "threshold", "value", "n_samples"))
    return {"ranks": P, "backend": "local-threads (one GPU)", "ms_per_fit": dt_s / steps * 1e3,
            "identical_to_dt_fit": bool(same), "timing": "host wall clock around synchronised fits"}


def extra_configs(args, dev, stream, rank=0, world=1):
    """BASELINE configs[0] (paper-sized LOO, rank 0) and configs[4] (hyper-parameter grid,
    the 16 min_samples_leaf fits spread over the ranks)."""
    import numpy as np
    import torch

    import datagen
    import paper_conf_ipps_metzgd23_b200 as dt
    out = {}
    # configs[0]: 40 rows (20 Table I CNNs x V100S / GTX 1080Ti) x 4 features, unlimited
    # depth, leave-one-out; the paper's DT accuracy is context, not a target
    gather = None
    if world > 1:
        import torch.distributed as dist

        def gather(obj):
            lst = [None] * world
            dist.all_gather_object(lst, obj)
            return lst
    X, y = datagen.paper_table(0)
    Xd, yd = torch.from_numpy(X).to(dev), torch.from_numpy(y).to(dev)
    for _ in range(3):
        yh = dt.dt_loo(Xd, yd, -1, 1)
    torch.cuda.synchronize()
    reps = 20
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record(stream)
    for _ in range(reps):
        yh = dt.dt_loo(Xd, yd, -1, 1)
    b.record(stream)
    torch.cuda.synchronize()
    m = dt.dt_eval(yd, yh, 4)
    out["c1_loo"] = {"workload": "configs[0]: 40 x 4 paper table, max_depth -1, LOO (40 refits)",
                     "us_per_loo": a.elapsed_time(b) / reps * 1e3, "mape": m["mape"], "r2": m["r2"],
                     "adj_r2": m["adj_r2"],
                     "paper_context": {"mape": 0.0573, "r2": 0.45, "adj_r2": 0.19,
                                       "note": "paper's private data (P:216); synthetic here"}}
    # configs[4]: 10M x 16 (seed 5), 70/30 hash split, max_depth 1..16 x min_samples_leaf 2^0..2^15
    n5 = args.grid_rows
    if n5 > 0:
        X5, y5 = dt.dt_gen_table(5, n5, d=16, device=dev)
        hold = torch.from_numpy(datagen.holdout_mask(5, n5)).to(dev)
        Xt, yt = X5[~hold].contiguous(), y5[~hold].contiguous()
        Xv, yv = X5[hold].contiguous(), y5[hold].contiguous()
        depths, ms = list(range(1, 17)), [1 << k for k in range(16)]
        # warm-up: the same grid (same shapes: workspace sizes, pooled memory)
        t0 = time.perf_counter()
        dt.grid_search(Xt, yt, Xv, yv, depths, ms, rank=rank, world=world, gather=gather)
        torch.cuda.synchronize()
        warm_ms = (time.perf_counter() - t0) * 1e3
        barrier(world)
        ga, gb = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        ga.record(stream)
        res, evals = dt.grid_search(Xt, yt, Xv, yv, depths, ms, rank=rank, world=world, gather=gather)
        gb.record(stream)
        torch.cuda.synchronize()
        ms_grid = max_over_ranks(ga.elapsed_time(gb), world)  # device time, max over ranks
        best = min(res.items(), key=lambda kv: kv[1][0])
        out["c5_grid"] = {"workload": f"configs[4]: {n5} x 16 (seed 5), 70/30 hash split, "
                                      "max_depth 1..16 x min_samples_leaf 2^0..2^15 = 256 fits",
                          "method": "dt_fit_grid: one presort, 16 deep level loops (one per m, spread over the "
                                    "ranks) + one fused all-depth held-out eval each",
                          "ranks": world, "timing": "CUDA events around the second identical grid run",
                          "ms": ms_grid, "warmup_ms_host": warm_ms, "split_evals_performed": evals,
                          "split_evals_per_s_performed": evals / (ms_grid / 1e3),
                          "best": {"max_depth": best[0][0], "min_samples_leaf": best[0][1],
                                   "mape": best[1][0], "r2": best[1][1]}}
        del X5, y5, Xt, yt, Xv, yv
    return out


def c3_measure(args, world, rank, dev, stream):
    """BASELINE configs[2]: 100M x 32 (S32, seed 3), max_depth 16, min_samples_leaf 1.
    N=1: dt_fit on one B200 (~110 GB of HBM: the level lists, double-buffered, hold the
    presort buffers) -- the strong-scaling reference of the N>1 headline.  Device-timed
    with CUDA events on the fit's stream; the first fit (planning + graph capture) is
    untimed.  One extra profiled fit splits presort / levels."""
    import torch

    import paper_conf_ipps_metzgd23_b200 as dt
    n, d, depth = args.c3_rows, 32, 16
    dt.dt_release_workspace()
    torch.cuda.empty_cache()
    X, y = dt.dt_gen_table(3, n, d=d, cnn_pool_bits=22, gpu_pool_bits=12, device=dev)
    def fit():
        return dt.dt_fit(X, y, depth, 1)
    tree = fit()
    reps = 3
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    barrier(world)
    torch.cuda.synchronize()
    a.record(stream)
    for _ in range(reps):
        tree = fit()
    b.record(stream)
    torch.cuda.synchronize()
    t = max_over_ranks(a.elapsed_time(b) / 1e3 / reps, world)
    # one profiled fit (direct enqueue) for the presort / level split; the cached graph
    # plan's buffers are released first (the direct path allocates its own)
    dt.dt_release_workspace()
    dt.dt_profile_reset()
    dt.dt_profile_enable(True)
    fit()
    dt.dt_profile_enable(False)
    prof = dt.dt_profile()
    dt.dt_release_workspace()
    del X, y
    torch.cuda.empty_cache()
    presort = sum(v["ms"] for k, v in prof.items() if k.startswith("presort"))
    levels = sum(v["ms"] for k, v in prof.items() if not k.startswith("presort"))
    return {"workload": f"configs[2]: {n} x {d} (S32, seed 3, pools 2^22 x 2^12), max_depth {depth}, min_samples_leaf 1",
            "mode": "dt_fit (1 GPU)",
            "ms_per_fit": t * 1e3, "split_evals_per_fit": tree.split_evals,
            "split_evals_per_s": tree.split_evals / t, "tree_nodes": tree.size, "tree_depth": tree.depth,
            "profiled_fit_ms": {"presort": presort, "levels": levels},
            "timing": "CUDA events around 3 fits after 1 untimed, max over ranks"}


def run_ours(args, world, rank, local):
    import torch

    import paper_conf_ipps_metzgd23_b200 as dt

    dev = torch.device("cuda", local)
    torch.cuda.set_device(dev)
    stream = torch.cuda.current_stream()
    # inputs resident in HBM (device generator, bit-identical to datagen)
    X, y = dt.dt_gen_table(1 + rank, N_TRAIN, d=D, device=dev)
    Xv, yv = dt.dt_gen_table(2 + 1000 * rank, N_TRAIN, d=D, device=dev)
    flush = torch.empty(256 * 1024 * 1024 // 4, dtype=torch.float32, device=dev)
    torch.cuda.synchronize()

    def step():
        tree = dt.dt_fit(X, y, MAX_DEPTH, MIN_LEAF)
        m = dt.dt_predict_eval(tree, Xv, yv, D)
        return tree, m

    for _ in range(args.warmup):
        tree, m = step()
    ev0 = [torch.cuda.Event(enable_timing=True) for _ in range(args.steps)]
    ev1 = [torch.cuda.Event(enable_timing=True) for _ in range(args.steps)]
    # ---- timed steps (headline): no profiling, so bounded-depth fits replay their
    # cached CUDA graph (the library's normal fast path)
    dt.dt_profile_enable(False)
    launches0 = dt.dt_launch_count()
    evals = 0
    with ClockSampler(local) as clk:
        barrier(world)
        torch.cuda.synchronize()
        for i in range(args.steps):
            flush.zero_()
            ev0[i].record(stream)
            tree, m = step()
            ev1[i].record(stream)
            evals += tree.split_evals
        torch.cuda.synchronize()
        barrier(world)
    launches = dt.dt_launch_count() - launches0
    ms = [a.elapsed_time(b) for a, b in zip(ev0, ev1)]
    t_total = sum(ms) / 1e3
    t_max = max_over_ranks(t_total, world)
    evals_all = sum_over_ranks(float(evals), world)
    value = evals_all / t_max
    step_ms = sum(ms) / len(ms)

    # ---- profiled steps (roofline): per-kernel CUDA events recorded by the library on
    # its stream, live in this process; the fit keeps its CUDA-graph replay (the graph is
    # captured once with event-record nodes around each kernel group: untimed warm-up)
    nprof = max(3, min(args.steps, 10))
    dt.dt_profile_enable(True, graph=True)
    step()
    torch.cuda.synchronize()
    dt.dt_profile_reset()
    pe0, pe1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    prof_ms = 0.0
    for _ in range(nprof):
        flush.zero_()
        pe0.record(stream)
        step()
        pe1.record(stream)
        torch.cuda.synchronize()
        prof_ms += pe0.elapsed_time(pe1)
    dt.dt_profile_enable(False)
    prof = dt.dt_profile()

    # roofline of the dominant kernel (largest device time inside the profiled steps)
    peak, peak_src = peaks()
    fit_kinds = {k: v for k, v in prof.items() if v["alg_bytes"] > 0}
    dom = max(fit_kinds, key=lambda k: fit_kinds[k]["ms"])
    d_ms = fit_kinds[dom]["ms"]
    achieved = fit_kinds[dom]["alg_bytes"] / (d_ms / 1e3) / 1e9
    traffic = None
    tpath = os.path.join(ROOT, "profiles", "traffic.json")
    if os.path.exists(tpath):
        with open(tpath) as fh:
            traffic = json.load(fh).get(dom)
    share = {k: round(v["ms"] / prof_ms, 4) for k, v in prof.items()}
    # every kernel kind with algorithmic bytes (the north star names scan, partition and
    # predict): achieved GB/s over its launches and the fraction of the measured peak
    by_kernel = {k: {"achieved_gbs": round(v["alg_bytes"] / (v["ms"] / 1e3) / 1e9, 1),
                     "frac": round(v["alg_bytes"] / (v["ms"] / 1e3) / 1e9 / peak, 4),
                     "ms_per_step": round(v["ms"] / nprof, 4)}
                 for k, v in fit_kinds.items()}
    roofline = {"bound": "hbm", "kernel": dom, "achieved": achieved, "peak": peak, "unit": "GB/s",
                "frac": achieved / peak, "peak_source": peak_src,
                "alg_bytes_per_launch": fit_kinds[dom]["alg_bytes"] / fit_kinds[dom]["launches"],
                "avg_launch_ms": d_ms / fit_kinds[dom]["launches"], "traffic": traffic,
                "measured": f"{nprof} profiled steps (ms/step {prof_ms / nprof:.3f}; unprofiled {step_ms:.3f}), "
                            "CUDA events recorded by event-record nodes inside the replayed fit graph around each kernel group",
                "by_kernel": by_kernel}

    # ---- e2e: through the C ABI with host buffers (pinned), H2D + D2H inside the region.
    # Every step copies its inputs from pinned host memory and reads the tree and the
    # metrics back.  Double-buffered: step i+1's inputs travel on a copy stream while
    # step i fits (the library keeps one cached graph per input buffer, two plans).
    Xh, yh = X.cpu().pin_memory(), y.cpu().pin_memory()
    Xvh, yvh = Xv.cpu().pin_memory(), yv.cpu().pin_memory()
    bufs = [tuple(torch.empty_like(t) for t in (X, y, Xv, yv)) for _ in range(2)]
    side = torch.cuda.Stream()
    h2d = sum(t.numel() * t.element_size() for t in (Xh, yh, Xvh, yvh))
    d2h = 0
    e_evals = 0

    def upload(buf):
        for dst, src in zip(buf, (Xh, yh, Xvh, yvh)):
            dst.copy_(src, non_blocking=True)

    # untimed warm-up of the e2e path (each buffer gets its cached fit graph)
    for buf in bufs:
        upload(buf)
        dt.dt_predict_eval(dt.dt_fit(buf[0], buf[1], MAX_DEPTH, MIN_LEAF), buf[2], buf[3], D)
    torch.cuda.synchronize()
    barrier(world)
    t0 = time.perf_counter()
    ready = [None, None]
    with torch.cuda.stream(side):
        upload(bufs[0])
        ready[0] = side.record_event()
    for i in range(args.e2e_steps):
        c, nx = i % 2, (i + 1) % 2
        if i + 1 < args.e2e_steps:
            side.wait_event(stream.record_event())  # buffer nx's previous step is done
            with torch.cuda.stream(side):
                upload(bufs[nx])
                ready[nx] = side.record_event()
        stream.wait_event(ready[c])
        Xd, yd, Xvd, yvd = bufs[c]
        tr = dt.dt_fit(Xd, yd, MAX_DEPTH, MIN_LEAF)   # returns the node array on the host
        mm = dt.dt_predict_eval(tr, Xvd, yvd, D)      # metrics to the host
        e_evals += tr.split_evals
        d2h = tr.size * 48 + 24
    torch.cuda.synchronize()
    e2e_t = max_over_ranks(time.perf_counter() - t0, world)
    e2e_value = sum_over_ranks(float(e_evals), world) / e2e_t
    del bufs

    # ---- DSE predictions/s (configs[3] shape on one GPU)
    dse = None
    if not args.no_dse:
        nd = 1 << args.dse_log2
        Xdse = dt.dt_gen_dse(3 + rank, 0, nd, 10, device=dev)
        tdse = dt.dt_fit(X, y, 20, 128)
        out = torch.empty(nd, dtype=torch.float64, device=dev)
        for _ in range(3):
            dt.dt_predict(tdse, Xdse, out=out)
        reps = 5
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        dt.dt_profile_reset()
        dt.dt_profile_enable(True)
        torch.cuda.synchronize()
        a.record(stream)
        for _ in range(reps):
            dt.dt_predict(tdse, Xdse, out=out)
        b.record(stream)
        torch.cuda.synchronize()
        dt.dt_profile_enable(False)
        pp = dt.dt_profile().get("predict")
        t = a.elapsed_time(b) / 1e3
        tmax = max_over_ranks(t, world)
        preds = sum_over_ranks(float(nd * reps), world) / tmax
        pach = pp["alg_bytes"] / (pp["ms"] / 1e3) / 1e9
        dse = {"predictions_per_s": preds, "candidates_per_rank": nd, "tree_nodes": tdse.size,
               "tree_depth": tdse.depth, "ms_per_pass": t / reps * 1e3,
               "roofline": {"bound": "hbm", "kernel": "predict", "achieved": pach, "peak": peak,
                            "unit": "GB/s", "frac": pach / peak,
                            "alg_bytes_per_launch": pp["alg_bytes"] / pp["launches"]}}
        del Xdse, out
        # factored DSE: the full configs[3] cross product, 2^20 CNNs x
        # 2^10 GPU configs = 2^30 candidates, composed on the fly from the two tables
        import datagen
        n_cnn, n_gpu = 1 << 20, 1 << 10
        cnn, gpu, src = datagen.dse_tables(3 + rank, 0, n_cnn, n_gpu)
        cnn_d, gpu_d = torch.from_numpy(cnn).to(dev), torch.from_numpy(gpu).to(dev)
        out = torch.empty(n_cnn * n_gpu, dtype=torch.float64, device=dev)
        for _ in range(3):
            dt.dt_predict_dse(tdse, cnn_d, gpu_d, src, out=out)
        torch.cuda.synchronize()
        dt.dt_profile_reset()
        dt.dt_profile_enable(True)
        a.record(stream)
        for _ in range(reps):
            dt.dt_predict_dse(tdse, cnn_d, gpu_d, src, out=out)
        b.record(stream)
        torch.cuda.synchronize()
        dt.dt_profile_enable(False)
        pp = dt.dt_profile().get("predict")
        t = a.elapsed_time(b) / 1e3
        tmax = max_over_ranks(t, world)
        fpreds = sum_over_ranks(float(n_cnn * n_gpu * reps), world) / tmax
        fach = pp["alg_bytes"] / (pp["ms"] / 1e3) / 1e9
        dse["factored"] = {
            "workload": "configs[3]: 2^20 CNNs x 2^10 GPU configs = 2^30 candidates per rank, "
                        "composed from the two tables (dt_predict_dse), same tree",
            "predictions_per_s": fpreds, "ms_per_pass": t / reps * 1e3,
            "roofline": {"bound": "hbm", "kernel": "predict_dse", "achieved": fach, "peak": peak,
                         "unit": "GB/s", "frac": fach / peak,
                         "alg_bytes_per_launch": pp["alg_bytes"] / pp["launches"],
                         "note": "8 B yhat write per prediction; the traversal is issue-bound"}}
        del out, cnn_d, gpu_d

    # ---- optional (--sharded-local P): the C2 table row-sharded over P host-thread ranks on this GPU
    sharded = None
    if world == 1 and args.sharded_local > 1:
        try:
            sharded = sharded_fit_measure(args, rank, dev, X, y, stream)
        except Exception as e:  # never let the extra measurement kill the headline
            sharded = {"error": f"{type(e).__name__}: {e}"}

    extra = None
    if not args.no_extra:
        try:
            extra = extra_configs(args, dev, stream, rank, world)
        except Exception as e:
            extra = {"error": f"{type(e).__name__}: {e}"}

    # ---- Random Forest: 16 bagged trees of the configs[1] table
    forest = None
    if not args.no_extra:
        try:
            T = 16
            # earlier sections leave cached fit plans (up to 2, e.g. the C5 grid's 10M-row
            # workspace); start from a clean pool so the timed forest holds only its own
            dt.dt_release_workspace()
            torch.cuda.empty_cache()
            fo = dt.dt_forest_fit(X, y, 2, MAX_DEPTH, MIN_LEAF, seed=1)  # warm-up (plans the graph)
            torch.cuda.synchronize()
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            barrier(world)
            a.record(stream)
            fo = dt.dt_forest_fit(X, y, T, MAX_DEPTH, MIN_LEAF, seed=1)
            b.record(stream)
            torch.cuda.synchronize()
            tf = max_over_ranks(a.elapsed_time(b) / 1e3, world)
            outv = torch.empty(Xv.shape[0], dtype=torch.float64, device=dev)
            dt.dt_forest_predict(fo, Xv, out=outv)
            torch.cuda.synchronize()
            a.record(stream)
            for _ in range(5):
                dt.dt_forest_predict(fo, Xv, out=outv)
            b.record(stream)
            torch.cuda.synchronize()
            tp = a.elapsed_time(b) / 1e3 / 5
            mf = dt.dt_eval(yv, outv, D)
            forest = {"workload": f"{T} bagged trees (bootstrap seed 1) of the configs[1] table, depth "
                                  f"{MAX_DEPTH}; predict + eval on the 1M held-out rows",
                      "split_evals_per_s": sum_over_ranks(float(fo.split_evals), world) / tf,
                      "ms_per_forest_fit": tf * 1e3, "predict_ms": tp * 1e3,
                      "predictions_per_s": Xv.shape[0] / tp, "eval_mape": mf["mape"], "eval_r2": mf["r2"]}
            del fo, outv
        except Exception as e:
            forest = {"error": f"{type(e).__name__}: {e}"}

    # ---- KNN regression: 2^16 training rows of the configs[1] table,
    # 2^20 queries (held-out rows), k = 5 (sklearn default); fp64 CUDA-core brute force
    knn = None
    if not args.no_extra:
        try:
            ntr = 1 << 16
            Xtr, ytr = X[:ntr].contiguous(), y[:ntr].contiguous()
            Xq = Xv[:1 << 20].contiguous()
            nqk = Xq.shape[0]  # the held-out rows (1M)
            outk = torch.empty(nqk, dtype=torch.float64, device=dev)
            dt.dt_knn_predict(Xtr, ytr, Xq[:4096], 5, out=outk[:4096])  # warm-up
            torch.cuda.synchronize()
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record(stream)
            dt.dt_knn_predict(Xtr, ytr, Xq, 5, out=outk)
            b.record(stream)
            torch.cuda.synchronize()
            tk = a.elapsed_time(b) / 1e3
            pairs = float(ntr) * nqk
            # fp64 pipe: 64 lanes / SM / clock (B200 FP64 37 TFLOPS = 2 x 64 x 148 x 1.965 GHz),
            # 2 instructions (DSUB, DFMA) per (query, row, feature)
            ops = 2.0 * D * pairs
            peak_ops = 64.0 * 148 * 1.965e9
            knn = {"workload": f"{ntr} training rows (configs[1] table) x {nqk} queries (held-out rows), "
                               f"d {D}, k 5", "ms": tk * 1e3, "distance_pairs_per_s": pairs / tk,
                   "predictions_per_s": nqk / tk,
                   "roofline": {"bound": "alu", "kernel": "knn (fp64 pipe)", "achieved": ops / tk / 1e12,
                                "peak": peak_ops / 1e12, "unit": "T fp64 instr/s",
                                "frac": ops / tk / peak_ops,
                                "peak_source": "derived: 64 fp64 lanes/SM/clk x 148 SMs x 1.965 GHz"}}
            del outk, Xtr, ytr, Xq
        except Exception as e:
            knn = {"error": f"{type(e).__name__}: {e}"}

    c3 = None
    if args.c3_rows > 0:
        del Xd, yd, Xvd, yvd
        try:
            c3 = c3_measure(args, world, rank, dev, stream)
        except Exception as e:
            c3 = {"error": f"{type(e).__name__}: {e}"}

    # ---- CPU baseline: the oracle on the host (rank 0, N=1 only)
    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu:
        rate, secs, ev, sk = oracle_rate(CPU_SAMPLE_ROWS)
        cpu = {"value": rate, "unit": "split evals/s", "cores": 1, "kind": "oracle",
               "sample": f"oracle fit on the first {CPU_SAMPLE_ROWS} of the {N_TRAIN} rows "
                         f"(seed 1), depth {MAX_DEPTH}: {ev} split evals in {secs:.1f} s",
               "cpu_model": _cpu_model(), "host_cores_available": os.cpu_count(),
               "pinned": "one core (sched_setaffinity)", "sklearn": sk}

    if rank == 0:
        if dse is not None:  # the prediction kernels' rooflines beside the fit's (north star:
            # split search AND prediction against HBM)
            roofline["predict"] = dict(dse["roofline"], workload="2^%d materialised DSE candidates" % args.dse_log2,
                                       predictions_per_s=dse["predictions_per_s"])
            if "factored" in dse:
                roofline["predict_dse_factored"] = dict(dse["factored"]["roofline"],
                                                        predictions_per_s=dse["factored"]["predictions_per_s"])
        line = {"metric": METRIC, "value": value, "unit": "split evals/s", "n_gpus": world,
                "steps": args.steps, "warmup": args.warmup, "ms_per_step": step_ms,
                "higher_is_better": True, "scaling": "weak", "vs_baseline": None,
                "dtype": "f64", "data": "synthetic", "config": workload_config(world),
                "e2e": {"value": e2e_value, "unit": "split evals/s", "h2d_bytes_per_step": h2d,
                        "d2h_bytes_per_step": d2h, "steps": args.e2e_steps},
                "gpu_launches": launches,
                "roofline": roofline, "cpu_baseline": cpu, "dse": dse, "sharded_fit": sharded, "extra_configs": extra,
                "c3_fit": c3, "forest": forest, "knn": knn,
                "clocks": clk.summary(),
                "fit": {"split_evals_per_step": evals // args.steps, "tree_nodes": tree.size,
                        "tree_depth": tree.depth, "eval_mape": m["mape"], "eval_r2": m["r2"],
                        "kernel_share_of_profiled_step": share,
                        "kernel_ms_per_step": {k: v["ms"] / nprof for k, v in prof.items()}}}
        print(json.dumps(line), flush=True)


def run_sharded(args, world, rank, local):
    """N>1 headline: BASELINE configs[2] (100M x 32, S32 seed 3, depth 16, m 1) as ONE fit
    row-sharded over the ranks (dt_fit_sharded over NCCL); rank r generates and holds rows
    [r n / N, (r + 1) n / N).  Strong scaling: value = the fit's split evals / the max over
    ranks of the device time per fit.  e2e: the same fit with the rank's rows copied from
    pinned host memory every step (H2D inside the timed region) and the tree read back."""
    import torch
    import torch.distributed as dist

    import paper_conf_ipps_metzgd23_b200 as dt
    dev = torch.device("cuda", local)
    torch.cuda.set_device(dev)
    stream = torch.cuda.current_stream()
    n, d, depth = args.c3_rows if args.c3_rows > 0 else 100_000_000, 32, 16
    lo, hi = rank * n // world, (rank + 1) * n // world
    X, y = dt.dt_gen_table(3, hi - lo, d=d, row0=lo, cnn_pool_bits=22, gpu_pool_bits=12, device=dev)

    def bcast(obj):
        lst = [obj]
        dist.broadcast_object_list(lst, src=0)
        return lst[0]
    comm = dt.dt_comm_init_nccl(rank, world, bcast)

    def fit(Xl, yl):
        return dt.dt_fit_sharded(comm, Xl, yl, lo, n, depth, 1, stream=stream)

    for _ in range(max(1, args.warmup)):
        tree = fit(X, y)
    steps = max(1, args.steps)
    ev0 = [torch.cuda.Event(enable_timing=True) for _ in range(steps)]
    ev1 = [torch.cuda.Event(enable_timing=True) for _ in range(steps)]
    launches0 = dt.dt_launch_count()
    with ClockSampler(local) as clk:
        barrier(world)
        torch.cuda.synchronize()
        for i in range(steps):
            ev0[i].record(stream)
            tree = fit(X, y)
            ev1[i].record(stream)
        torch.cuda.synchronize()
        barrier(world)
    launches = dt.dt_launch_count() - launches0
    t_total = sum(a.elapsed_time(b) for a, b in zip(ev0, ev1)) / 1e3
    t_max = max_over_ranks(t_total, world)
    evals = tree.split_evals  # the global tree's split evals (same on every rank)
    value = evals * steps / t_max
    # e2e: host rows -> device every step, the tree back to the host
    Xh, yh = X.cpu().pin_memory(), y.cpu().pin_memory()
    Xd, yd = torch.empty_like(X), torch.empty_like(y)
    e_steps = max(1, min(args.e2e_steps, steps))
    barrier(world)
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    for _ in range(e_steps):
        Xd.copy_(Xh, non_blocking=True)
        yd.copy_(yh, non_blocking=True)
        tr = fit(Xd, yd)
    torch.cuda.synchronize()
    e2e_t = max_over_ranks(time.perf_counter() - t0, world)
    # per-kernel roofline of this rank's fused pass (one profiled fit)
    peak, peak_src = peaks()
    dt.dt_profile_reset()
    dt.dt_profile_enable(True)
    fit(X, y)
    dt.dt_profile_enable(False)
    prof = dt.dt_profile()
    roof = None
    fk = {k: v for k, v in prof.items() if v["alg_bytes"] > 0}
    if fk:
        dom = max(fk, key=lambda k: fk[k]["ms"])
        ach = fk[dom]["alg_bytes"] / (fk[dom]["ms"] / 1e3) / 1e9
        roof = {"bound": "hbm", "kernel": dom, "achieved": ach, "peak": peak, "unit": "GB/s", "frac": ach / peak,
                "peak_source": peak_src, "alg_bytes_per_launch": fk[dom]["alg_bytes"] / fk[dom]["launches"],
                "avg_launch_ms": fk[dom]["ms"] / fk[dom]["launches"], "traffic": None,
                "measured": "rank 0, one profiled sharded fit, per-launch CUDA events",
                "by_kernel_ms_per_fit": {k: round(v["ms"], 3) for k, v in prof.items()}}
    if rank == 0:
        line = {"metric": METRIC, "value": value, "unit": "split evals/s", "n_gpus": world, "steps": steps,
                "warmup": args.warmup, "ms_per_step": t_max / steps * 1e3, "higher_is_better": True,
                "scaling": "strong", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
                "config": {"workload": f"configs[2]: {n} x {d} (S32, seed 3, pools 2^22 x 2^12), max_depth {depth}, "
                                       "min_samples_leaf 1; one fit row-sharded over the ranks",
                           "n_train": n, "d": d, "max_depth": depth, "min_samples_leaf": 1,
                           "parallelism": f"rowshard{world}", "ranks": world,
                           "l2": "inputs (12.8 GB of X) larger than L2"},
                "e2e": {"value": evals * e_steps / e2e_t, "unit": "split evals/s",
                        "h2d_bytes_per_step": (hi - lo) * (4 * d + 8) * world, "d2h_bytes_per_step": tr.size * 48,
                        "steps": e_steps},
                "gpu_launches": launches, "roofline": roof, "cpu_baseline": None,
                "fit": {"split_evals_per_fit": evals, "tree_nodes": tree.size, "tree_depth": tree.depth},
                "clocks": clk.summary()}
        print(json.dumps(line), flush=True)


def relaunch(args):
    """--gpus N without a torchrun environment: re-run this script under
    torch.distributed.run with N processes on this node (127.0.0.1 rendezvous)."""
    import socket
    sk = socket.socket()
    sk.bind(("127.0.0.1", 0))
    port = sk.getsockname()[1]
    sk.close()
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
           "--master-addr", "127.0.0.1", "--master-port", str(port), os.path.abspath(__file__)] + sys.argv[1:]
    os.execv(sys.executable, cmd)


def main():
    args = parse()
    if args.gpus > 1 and "WORLD_SIZE" not in os.environ:
        relaunch(args)
    world, rank, local = dist_init()
    if args.impl == "reference":
        run_reference(args, world, rank)
    elif world > 1 or args.force_sharded:
        run_sharded(args, world, rank, local)
    else:
        run_ours(args, world, rank, local)
    if world > 1:
        import torch.distributed as dist
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
