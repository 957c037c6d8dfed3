"""Benchmark of the mSTAMP hot path (BASELINE.json metric: d*n^2 matrix-profile cells*dims/s).

A "step" = one whole pass of the hot path (precompute -> fused diagonal kernel ->
finalize) over the workload, inputs resident in HBM.  BASELINE.json's metric names no
configuration, so the headline runs the largest single-GPU config, C3 (self-join, d=64,
n=262144, m=256, seeded random walk + planted motif), in FP32; Mixed, FP16 and FP64 are timed
on the same workload under "per_precision", C2 (d=16) is reported as context, and one
diagonal band of C4 / C5 at full input size under "per_config_band".  With --gpus N > 1 the
default workload is C4 (AB-join d=128, n=2^20, m=256), the config BASELINE names for
1/2/4/8 GPUs.

  python bench.py [--gpus N] [--steps K] [--warmup W] [--precision fp32] [--config C2]
  python bench.py --impl reference ...   (the FP64 CPU oracle on host cores, sampled rows)

Multi-GPU (torchrun, one process per GPU): each rank computes its equal-cell diagonal
band, one NCCL MINLOC all-reduce merges the partial profiles (the path's only exchange);
time = max over ranks, value = total d*n^2 / time ("scaling": "strong": the job is
fixed, bands shrink with N).
"""
from __future__ import annotations

import argparse
import json
import math
import os
import statistics
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

from paper_conf_ipps_juryl022_b200 import datagen  # noqa: E402

PEAKS_PATH = os.path.join(ROOT, "MEASURED_PEAKS.json")
METRIC = "matrix-profile cells*dims/sec (d*n^2/s)"
UNIT = "cells*dims/s"
SM_COUNT = 148
ALU_LANES = 64          # ALU-pipe lanes per SM per clock (FMNMX/FSETP/FSEL), B300_MICROARCH "alu rt=2/SMSP"
NOMINAL_SM_MHZ = 1965.0
PIPE_PEAKS_PATH = os.path.join(os.path.dirname(os.path.abspath(__file__)), "profiles", "r1_pipe_peaks.json")


def alu_lanes():
    """ALU-pipe lanes per SM per clock: measured by scripts/pipe_peaks.cu on a B200 (FMNMX with
    8 independent chains per thread, 2048 threads/SM), else the nominal 64."""
    try:
        with open(PIPE_PEAKS_PATH) as f:
            return float(json.load(f)["fmnmx_alu"]["lanes_per_sm_clk"]), "measured"
    except (OSError, KeyError, ValueError):
        return float(ALU_LANES), "nominal"


def alu_peak_ops(sm_mhz=None):
    lanes, _ = alu_lanes()
    return SM_COUNT * lanes * (sm_mhz or NOMINAL_SM_MHZ) * 1e6


def in_memory_bytes(d, n, m, prec, self_join):
    """Device bytes of the in-memory path's per-position arrays (stats, pair format, seed
    operands, keys, window-stat scratch) and P / I: what mp_compute_stream bounds."""
    half = prec in ("fp16", "mixed", "fp16c", "fp16ck")
    sb = 16 if half else (32 if prec == "fp64" else 16)
    tb = 8 if prec == "fp64" else (2 if prec in ("fp16", "fp16c") else 4)
    dp = 1 << (d - 1).bit_length()
    side = n * d * sb + (n + 1) * d * 16 * half + (n + m - 1) * dp * tb + n * dp * tb + 2 * n * d * (8 if prec == "fp32" else tb)
    keys = n * d * (16 if prec == "fp64" else 8)
    return int(side * (1 if self_join else 2) + keys + 16 * d * n)


def batcher_ce(N: int) -> int:
    """Comparators of Batcher's odd-even merge sort network on N inputs (as sort_net builds it)."""
    c = 0
    p = 1
    while p < N:
        k = p
        while k >= 1:
            j = k % p
            while j + k < N:
                for i in range(k):
                    if i + j + k < N and (i + j) // (2 * p) == (i + j + k) // (2 * p):
                        c += 1
                j += 2 * k
            k >>= 1
        p <<= 1
    return c


def alu_ops_per_cell_dim(d: int, self_join: bool) -> float:
    """Algorithmic ALU-pipe ops per computed cell*dim: clamp 1 + the d-way sort
    network (2 min/max per Batcher comparator, padded to a power of two, per dim) + the
    min-update, 3 per profile side (row; + column for the self-join): 9.5 / 14.9 / 24 / 27 / 37
    for C1..C5.  This is the roofline's op count."""
    dp = 1
    while dp < d:
        dp <<= 1
    return 1.0 + 2.0 * batcher_ce(dp) / d + 3.0 * (2.0 if self_join else 1.0)


def alu_ops_filtered(d: int, self_join: bool) -> float:
    """The same count for the filtered design the kernels implement (no clamp: |.| is a free
    operand modifier; one threshold compare per side instead of the 3-op min-update; the
    update itself runs on the rare cells that pass): a second, stricter figure."""
    dp = 1
    while dp < d:
        dp <<= 1
    return 2.0 * batcher_ce(dp) / d + (2.0 if self_join else 1.0)


def computed_cells(n: int, e: int, self_join: bool) -> int:
    if self_join:
        k = n - e - 1
        return k * (k + 1) // 2 if k > 0 else 0
    return n * n


class ClockSampler:
    """nvidia-smi clocks / throttle reasons sampled during the timed region."""

    Q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.hw_slowdown,"
         "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
         "clocks_event_reasons.sw_power_cap")

    def __init__(self, index: int):
        self.index = index
        self.proc = None
        self.lines = []
        self.t = None

    def start(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.Q}",
                                          "--format=csv,noheader,nounits", "-lms", "100"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except OSError:
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append(line.strip())

    def stop(self):
        if self.proc is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except subprocess.TimeoutExpired:
            self.proc.kill()
        self.t.join(timeout=2)
        sm, smax, reasons = [], [], set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for ln in self.lines:
            f = [x.strip() for x in ln.split(",")]
            if len(f) < 8:
                continue
            try:
                sm.append(float(f[1]))
                smax.append(float(f[2]))
            except ValueError:
                continue
            for nm, v in zip(names, f[4:8]):
                if v.lower().startswith("active"):
                    reasons.add(nm)
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(smax) if smax else None,
                "reasons": sorted(reasons), "samples": len(sm)}


def load_traffic(config, prec):
    try:
        with open(os.path.join(ROOT, "profiles", "traffic.json")) as f:
            return json.load(f).get(f"{config}/{prec}", {}).get("traffic_bytes")
    except (OSError, ValueError):
        return None


def load_peaks():
    try:
        with open(PEAKS_PATH) as f:
            return json.load(f), "measured"
    except OSError:
        return {"hbm_gbs": 6650.0, "bf16_tflops": 1590.0, "sm_max_mhz": NOMINAL_SM_MHZ}, "fallback"


def alu_ops_mode(d: int, self_join: bool, prec: str) -> float:
    """ALU-pipe ops per computed cell*dim by precision mode: FP32 and FP64 (whose common path is
    the FP32 filter: same sort, scan and compares) as alu_ops_per_cell_dim; FP16 / Mixed pack two
    cells in a half2, so each HMNMX2 / HSETP2 serves two cell*dims."""
    ops = alu_ops_per_cell_dim(d, self_join)
    return ops / 2.0 if prec in ("fp16", "mixed", "fp16c", "fp16ck") else ops


_PROBE_CACHE = {}


def band_probe(ctx, torch, dev, name: str, prec: str, target_cell_dims: float = 3e11, peak=None):
    """Throughput of one diagonal band of a larger BASELINE config at its full input size: the
    unit one rank computes under bench.py --gpus N (mp_partial_device), timed by the library's
    CUDA events around the main kernel.  The band is the middle one of a W-way equal-cell split
    sized to ~target_cell_dims computed cell*dims, so the probe takes seconds, not the minutes
    to hours of the full grid on one GPU."""
    from paper_conf_ipps_juryl022_b200 import mstamp
    if name not in _PROBE_CACHE:  # one synthetic input per config, resident across its probes
        _PROBE_CACHE.clear()
        torch.cuda.empty_cache()
        cfg = datagen.make(name)
        _PROBE_CACHE[name] = (cfg, torch.from_numpy(cfg["T"]).to(dev),
                              None if cfg["Tr"] is None else torch.from_numpy(cfg["Tr"]).to(dev))
    cfg, T, Tr = _PROBE_CACHE[name]
    d, n, m, e = cfg["d"], cfg["n"], cfg["m"], cfg["exclusion"]
    self_join = cfg["Tr"] is None
    total = computed_cells(n, e, self_join) * d
    W = max(1, int(round(total / target_cell_dims)))
    r = W // 2
    _, bc = mstamp.plan_bands(d, n, m, prec, e, self_join, W)
    keys = torch.empty(mstamp.key_words(d, n, prec), dtype=torch.int64, device=dev)
    kms = []
    for _ in range(2):  # the first launch also pays one-time setup; report the second
        ctx.partial_device(T, m, keys, r, W, prec, e, Tr=Tr)
        torch.cuda.synchronize()
        kms.append(ctx.last_timing()[0])
    del keys
    cd = int(bc[r]) * d
    rate = cd / (kms[-1] * 1e-3)
    peak = peak or alu_peak_ops()
    return {"workload": f"{'self' if self_join else 'AB'}-join d={d} n={n} m={m}", "precision": prec,
            "band": [r, W], "band_cell_dims": cd, "main_kernel_ms": kms[-1],
            "computed_cell_dims_per_s": rate, "alu_frac": rate * alu_ops_mode(d, self_join, prec) / peak,
            "full_grid_estimate_s_1gpu": total / rate}


def launches_per_step(prec: str, self_join: bool) -> int:
    # check_finite (1 per series) + precompute (pre_stats, pre_diff, pre_pm) per series
    # + init_keys + mp_diag + [keys64_to_ext] + finalize
    series = 1 if self_join else 2
    pre = 3
    return series * (1 + pre) + 1 + 1 + (1 if prec == "fp64" else 0) + 1


# ---------------------------------------------------------------------------- CPU oracle leg
def oracle_sample(cfg, target_s: float = 15.0, max_rows: int = 8192):
    """Time the FP64 oracle (as it stands) on sampled query rows of the workload.
    Returns (cell*dims per second, rows, seconds, threads, how).  Each sampled row is one query
    window against all n reference windows x d dims.  Small configs run oracle.mstamp (window
    statistics of the whole series once, then the rows); where those statistics alone would take
    longer than the sample (n d m > 2e9, C3..C5) the rows run oracle.mstamp_band over every
    diagonal, which computes each window's statistics where it needs them."""
    import oracle
    oracle.build()
    T, Tr, m, e, n, d = cfg["T"], cfg["Tr"], cfg["m"], cfg["exclusion"], cfg["n"], cfg["d"]
    threads = os.cpu_count() or 1
    rng = np.random.default_rng(0)
    big = n * d * m > 2e9
    how = "oracle.mstamp_band (all diagonals)" if big else "oracle.mstamp"

    def run(rows):
        if big:
            lo, hi = (0, n) if Tr is None else (-(n - 1), n)
            oracle.mstamp_band(T, m, rows, lo, hi, e, Tr=Tr, nthreads=threads)
        else:
            oracle.mstamp(T, m, e, Tr=Tr, rows=rows, nthreads=threads)

    rows = np.sort(rng.choice(n, size=min(threads, n), replace=False))
    t0 = time.perf_counter()
    run(rows)
    dt = time.perf_counter() - t0
    for _ in range(2):  # calibrate (the first call also pays the O(n d m) window stats)
        nr = int(min(max_rows, max(len(rows), len(rows) * target_s / max(dt, 1e-6))))
        nr = max(threads, (nr // threads) * threads)
        rows = np.sort(rng.choice(n, size=min(nr, n), replace=False))
        t0 = time.perf_counter()
        run(rows)
        dt = time.perf_counter() - t0
        if dt > 0.5 * target_s or nr >= max_rows:
            break
    cells = len(rows) * n * d          # each sampled row: all n reference windows x d dims
    return cells / dt, len(rows), dt, threads, how


def run_reference(args):
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return 0
    cfg = datagen.make(args.config)
    vals = []
    for _ in range(args.warmup):
        oracle_sample(cfg, target_s=2.0)
    meta = None
    for _ in range(args.steps):
        v, nr, dt, th, how = oracle_sample(cfg, target_s=args.ref_seconds)
        vals.append(v)
        meta = (nr, dt, th, how)
    value = statistics.mean(vals)
    line = {"impl": "reference", "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": meta[1] * 1e3,
            "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "f64",
            "data": "synthetic", "config": config_json(args, cfg),
            "cpu_baseline": {"value": value, "unit": UNIT, "cores": meta[2], "kind": "oracle",
                             "precision": "fp64",
                             "sample": f"{meta[0]} random query rows x all n reference windows per step ({meta[3]})"},
            "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)
    return 0


def config_json(args, cfg):
    return {"workload": f"{args.config}: {'self' if cfg['Tr'] is None else 'AB'}-join d={cfg['d']} "
                        f"n={cfg['n']} m={cfg['m']} exclusion={cfg['exclusion']}",
            "d": cfg["d"], "n": cfg["n"], "m": cfg["m"], "exclusion": cfg["exclusion"],
            "join": "self" if cfg["Tr"] is None else "ab", "precision": args.precision,
            "parallelism": f"diagonal-bands x{args.gpus}",
            "l2": "flushed between timed steps (256 MiB write)"}


# ---------------------------------------------------------------------------- GPU leg
def property_check(P, I, cfg):
    """Oracle-free checks of a (merged) profile at every (k, i): the distance bound
    0 <= P <= 2 sqrt(m), P non-decreasing in k, finite where an admissible j exists, and the
    planted motif found in its dimensions (I[k][a] = b).  Used for the multi-GPU merge, whose
    full 1-GPU recomputation would take minutes to hours at C4 / C5."""
    import torch
    m, d, n = cfg["m"], cfg["d"], cfg["n"]
    fin = torch.isfinite(P)
    ok_bound = bool(((P[fin] >= 0) & (P[fin] <= 2 * math.sqrt(m) * (1 + 1e-6))).all())
    diff = torch.diff(torch.where(fin, P, torch.zeros_like(P)), dim=0)
    ok_mono = bool((diff >= -1e-6 * torch.where(fin[1:], P[1:], torch.ones_like(P[1:]))).all())
    ok_idx = bool(((I[fin] >= 0) & (I[fin] < n)).all())
    pos = datagen.motif_positions(n, m)
    ok_motif = None
    if pos is not None:
        a, b = pos
        ok_motif = bool((I[: max(1, d // 2), a] == b).all())
    return {"bound": ok_bound, "monotone_in_k": ok_mono, "index_range": ok_idx, "planted_motif": ok_motif}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=3)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--precision", default="fp32")
    ap.add_argument("--config", default=None, help="C1..C5 (default: C3 at N = 1, C4 at N > 1)")
    ap.add_argument("--impl", default="native", choices=["native", "reference"])
    ap.add_argument("--ref-seconds", type=float, default=15.0)
    ap.add_argument("--no-per-precision", action="store_true")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-context", action="store_true", help="skip the C2 context line")
    ap.add_argument("--no-per-config", action="store_true",
                    help="skip the one-band throughput probes of the larger BASELINE configs")
    ap.add_argument("--merge-check", default="auto", choices=["auto", "full", "properties", "off"],
                    help="N > 1: 'full' recomputes the job on one GPU and compares bit for bit (C1/C2: "
                         "'auto'), 'properties' checks bound / monotonicity / planted motif (larger configs)")
    ap.add_argument("--backend", default="nccl", help="process-group backend for N>1 (gloo: functional "
                    "test of the multi-rank path, e.g. several ranks on one GPU via MP_BENCH_DEVICE)")
    ap.add_argument("--dry-run", action="store_true",
                    help="functional run of the multi-rank path: one step, no warm-up; the line says "
                         "dry_run and is not a bench value")
    ap.add_argument("--no-stream", action="store_true", help="skip the beyond-memory streaming leg")
    ap.add_argument("--stream-bytes", type=int, default=512 << 20,
                    help="device budget of the streaming leg (mp_compute_stream)")
    ap.add_argument("--per-precision", action="store_true",
                    help="N > 1: also time the other precisions (off by default: C4 FP64 takes minutes per step)")
    args = ap.parse_args()
    args.warmup = 0 if args.dry_run else max(args.warmup, 3)
    world0 = int(os.environ.get("WORLD_SIZE", "1"))
    if args.dry_run:
        args.steps = 1
        args.no_per_precision = args.no_context = args.no_per_config = args.no_cpu_baseline = True
        args.no_stream = True
    if world0 > 1 and not args.per_precision:
        args.no_per_precision = True
    world = int(os.environ.get("WORLD_SIZE", "1"))
    if args.config is None:
        args.config = "C3" if world == 1 else "C4"
    if args.impl == "reference":
        return run_reference(args)

    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("MP_BENCH_DEVICE", os.environ.get("LOCAL_RANK", "0")))
    if world > 1 and args.backend == "nccl":
        # NCCL init logging: the communicator's size and transport (NVLink / NVLS) go to stderr
        os.environ.setdefault("NCCL_DEBUG", "INFO")
        os.environ.setdefault("NCCL_DEBUG_SUBSYS", "INIT")
    import torch
    import torch.distributed as dist
    from paper_conf_ipps_juryl022_b200 import mstamp

    torch.cuda.set_device(local)
    if world > 1:
        if args.backend == "nccl":
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
        else:
            dist.init_process_group(args.backend)
    dev = torch.device("cuda", local)
    ctx = mstamp.Context(local)
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)
    stream = torch.cuda.current_stream(dev)

    def load_cfg(name):
        cfg = datagen.make(name)
        T = torch.from_numpy(cfg["T"]).to(dev)
        Tr = None if cfg["Tr"] is None else torch.from_numpy(cfg["Tr"]).to(dev)
        return cfg, T, Tr

    def runner(cfg, T, Tr, ctx=ctx):
        d, n, m, e = cfg["d"], cfg["n"], cfg["m"], cfg["exclusion"]
        P = torch.empty(d, n, dtype=torch.float64, device=dev)
        I = torch.empty(d, n, dtype=torch.int64, device=dev)
        keys = {}

        def one_step(prec):
            """One pass of the whole hot path; returns (device ms, main-kernel ms)."""
            flush.fill_(1)
            if world > 1:
                dist.barrier()
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            if world == 1:
                ctx.compute_device(T, m, P, I, prec, e, Tr=Tr, stream=stream)
            else:
                if prec not in keys:
                    keys[prec] = torch.empty(mstamp.key_words(d, n, prec), dtype=torch.int64, device=dev)
                k = keys[prec]
                ctx.partial_device(T, m, k, rank, world, prec, e, Tr=Tr, stream=stream)
                mstamp.merge_partials(ctx, k, d, n, prec)
                if rank == 0:
                    ctx.finalize_device(d, n, k, P, I, prec, stream=stream)
            e1.record(stream)
            torch.cuda.synchronize()
            kms, _ = ctx.last_timing()
            return e0.elapsed_time(e1), kms

        def timed(prec, steps, warm, sample_clocks=False):
            for _ in range(warm):
                one_step(prec)
            cs = ClockSampler(local) if sample_clocks else None
            if cs:
                cs.start()
                time.sleep(0.3)
            ms, kms = [], []
            for _ in range(steps):
                a, b = one_step(prec)
                ms.append(a)
                kms.append(b)
            clocks = cs.stop() if cs else None
            tot = torch.tensor([sum(ms)], dtype=torch.float64, device=dev)
            if world > 1:
                dist.all_reduce(tot, op=dist.ReduceOp.MAX)
            return tot.item() / steps, statistics.mean(kms), clocks

        return timed, P, I

    cfg, T, Tr = load_cfg(args.config)
    d, n, m, e = cfg["d"], cfg["n"], cfg["m"], cfg["exclusion"]
    self_join = cfg["Tr"] is None
    timed, Plast, Ilast = runner(cfg, T, Tr)
    ms, kms, clocks = timed(args.precision, args.steps, args.warmup, sample_clocks=True)
    run_mhz = (clocks or {}).get("sm_mhz") or NOMINAL_SM_MHZ
    dn2 = d * n * n
    value = dn2 / (ms * 1e-3)

    merge_check = None
    if world > 1:
        mode = args.merge_check
        if mode == "auto":
            mode = "full" if args.config in ("C1", "C2") else "properties"
        if rank == 0 and mode == "full":
            # outside the timed region: the merged N-rank result must equal the 1-GPU result bit
            # for bit (fixed tile plan, lexicographic MINLOC merge: DESIGN.md section 10)
            P1 = torch.empty(d, n, dtype=torch.float64, device=dev)
            I1 = torch.empty(d, n, dtype=torch.int64, device=dev)
            ctx.compute_device(T, m, P1, I1, args.precision, e, Tr=Tr, stream=stream)
            torch.cuda.synchronize()
            merge_check = {"bit_identical_to_1gpu": bool(torch.equal(P1, Plast) and torch.equal(I1, Ilast))}
            del P1, I1
        elif rank == 0 and mode == "properties":
            merge_check = property_check(Plast, Ilast, cfg)

    cells = computed_cells(n, e, self_join)
    peak_ops = alu_peak_ops(run_mhz)

    def frac(kms_, d_, cells_, self_, prec_):
        rate = cells_ * d_ / (kms_ * 1e-3)
        return rate * alu_ops_mode(d_, self_, prec_) / peak_ops

    per_prec = {}
    if not args.no_per_precision:
        for prec in ("fp32", "mixed", "fp16", "fp64"):
            if prec == args.precision:
                per_prec[prec] = {"value": value, "ms_per_step": ms, "main_kernel_ms": kms, "steps": args.steps}
            else:
                # FP64 takes ~50 s per C3 step: one warm-up, one timed step
                st, wu = (1, 1) if prec == "fp64" and d * n * n > 1e12 else (max(1, min(args.steps, 3)), 1)
                p_ms, p_kms, _ = timed(prec, st, wu)
                per_prec[prec] = {"value": dn2 / (p_ms * 1e-3), "ms_per_step": p_ms, "main_kernel_ms": p_kms,
                                  "steps": st}
            per_prec[prec]["alu_frac"] = frac(per_prec[prec]["main_kernel_ms"], d, cells, self_join, prec)
            per_prec[prec]["computed_cell_dims_per_s"] = cells * d / (per_prec[prec]["main_kernel_ms"] * 1e-3)
        # Mixed with tensor-core seeds (seed_mode MP_SEEDS_TC, NEXT-3): the seed GEMMs run inside
        # the timed step (main_kernel_ms spans the seed GEMMs and the fused-kernel chunks)
        if d >= 64:
            ctx_tc = mstamp.Context(local, seed_mode="tc")
            timed_tc, _, _ = runner(cfg, T, Tr, ctx_tc)
            p_ms, p_kms, _ = timed_tc("mixed", max(1, min(args.steps, 3)), 1)
            per_prec["mixed_tc_seeds"] = {"value": dn2 / (p_ms * 1e-3), "ms_per_step": p_ms, "main_kernel_ms": p_kms,
                                          "steps": max(1, min(args.steps, 3)),
                                          "alu_frac": frac(p_kms, d, cells, self_join, "mixed")}
            ctx_tc.close()
            del timed_tc

    context = None
    if not args.no_context and world == 1 and args.config != "C2":
        c2, T2, Tr2 = load_cfg("C2")
        timed2, _, _ = runner(c2, T2, Tr2)
        context = {"workload": "C2: self-join d=16 n=65536 m=128", "per_precision": {}}
        cells2 = computed_cells(c2["n"], c2["exclusion"], True)
        for prec in ("fp32", "mixed", "fp16", "fp64"):
            p_ms, p_kms, _ = timed2(prec, 3, 1)
            context["per_precision"][prec] = {
                "value": c2["d"] * c2["n"] ** 2 / (p_ms * 1e-3), "ms_per_step": p_ms, "main_kernel_ms": p_kms,
                "alu_frac": frac(p_kms, c2["d"], cells2, True, prec)}
        del T2, Tr2, timed2
        torch.cuda.empty_cache()

    per_cfg = {}
    if not args.no_per_config and world == 1:
        for name, prec in (("C4", "fp32"), ("C4", "mixed"), ("C4", "fp64"), ("C5", "fp32"), ("C5", "mixed"),
                           ("C5", "fp16"), ("C5", "fp64")):
            if name == args.config:
                continue
            per_cfg[f"{name}/{prec}"] = band_probe(ctx, torch, dev, name, prec, peak=peak_ops)
        _PROBE_CACHE.clear()
        torch.cuda.empty_cache()

    # e2e through the C-ABI host entry point (pinned host input and output buffers, H2D + D2H
    # inside the timed region)
    e2e = None
    if world == 1:
        Th = torch.from_numpy(cfg["T"]).pin_memory().numpy()
        Trh = None if self_join else torch.from_numpy(cfg["Tr"]).pin_memory().numpy()
        outs = (torch.empty((d, n), dtype=torch.float64, pin_memory=True).numpy(),
                torch.empty((d, n), dtype=torch.int64, pin_memory=True).numpy())
        ctx.compute(Th, m, args.precision, e, Tr=Trh, out=outs)
        ts = []
        for _ in range(args.steps):
            flush.fill_(1)
            torch.cuda.synchronize()
            t0 = time.perf_counter()
            ctx.compute(Th, m, args.precision, e, Tr=Trh, out=outs)
            ts.append(time.perf_counter() - t0)
        L = n + m - 1
        e2e = {"value": dn2 / statistics.mean(ts), "unit": UNIT,
               "h2d_bytes_per_step": d * L * 8 * (1 if self_join else 2), "d2h_bytes_per_step": 2 * d * n * 8,
               "ms_per_step": statistics.mean(ts) * 1e3}

    # beyond-memory streaming (mp_compute_stream, NEXT-4): the same job with a device budget far
    # below the in-memory footprint; host T in, host P / I out (timed like e2e), checked bit for
    # bit against the in-memory result of the e2e leg
    stream = None
    if world == 1 and not args.no_stream:
        Ps = (np.empty((d, n)), np.empty((d, n), dtype=np.int64))
        t0 = time.perf_counter()
        ctx.compute_stream(Th, m, args.precision, e, Tr=Trh, device_bytes=args.stream_bytes, out=Ps)
        dt = time.perf_counter() - t0
        R, Wb, peak, nl = ctx.last_stream_info()
        skms, _ = ctx.last_timing()
        stream = {"value": dn2 / dt, "unit": UNIT, "ms": dt * 1e3, "main_kernel_ms": skms,
                  "device_bytes": args.stream_bytes, "peak_mapped_bytes": peak, "rows_per_chunk": R,
                  "diagonals_per_band": Wb, "launches": nl,
                  "in_memory_device_bytes": in_memory_bytes(d, n, m, args.precision, self_join),
                  "bit_identical_to_in_memory": bool(np.array_equal(Ps[0], outs[0]) and np.array_equal(Ps[1], outs[1])),
                  "vs_e2e": (dn2 / dt) / e2e["value"] if e2e else None}
        del Ps

    if rank == 0:
        peaks, src = load_peaks()
        # roofline of the dominant kernel: algorithmic ops of the cells THIS launch computed (rank
        # 0's band when N > 1) over its CUDA-event duration
        band_cells = cells
        if world > 1:
            _, bc = mstamp.plan_bands(d, n, m, args.precision, e, self_join, world)
            band_cells = int(bc[0])
        ops = alu_ops_mode(d, self_join, args.precision) * band_cells * d
        lanes, lsrc = alu_lanes()
        peak_tops = peak_ops / 1e12
        achieved = ops / (kms * 1e-3) / 1e12 if kms > 0 else None
        kname = {"fp32": "mp_diag_ctab" if d > 32 else "mp_diag", "fp64": "mp_diag_cta64" if d > 32 else "mp_diag64f"}
        roof = {"bound": "alu", "achieved": achieved, "peak": peak_tops, "unit": "Tops/s",
                "frac": achieved / peak_tops if achieved else None,
                "traffic": load_traffic(args.config, args.precision),
                "kernel": kname.get(args.precision, "mp_diag_cta_h" if d > 32 else "mp_diag_h"),
                "ops_per_cell_dim": alu_ops_mode(d, self_join, args.precision),
                "ops_basis": "SURVEY 8(d): clamp 1 + 2 CE(d_pad)/d + 3 per profile side",
                "frac_filtered_ops": (alu_ops_filtered(d, self_join) * band_cells * d / (kms * 1e-3) / 1e12 / peak_tops
                                      / (2.0 if args.precision in ("fp16", "mixed", "fp16c", "fp16ck") else 1.0)) if kms > 0 else None,
                "computed_cell_dims": band_cells * d,
                "peak_basis": f"{SM_COUNT} SM x {lanes:.2f} FMNMX lanes/SM/clk ({lsrc}: scripts/pipe_peaks.cu -> "
                              f"profiles/r1_pipe_peaks.json; MEASURED_PEAKS {src} has no ALU figure) x {run_mhz:.0f} MHz "
                              "(SM clock sampled during the timed region)"}
        cpu = None
        if not args.no_cpu_baseline and world == 1:
            v, nr, dt, th, how = oracle_sample(cfg, target_s=args.ref_seconds)
            cpu = {"value": v, "unit": UNIT, "cores": th, "kind": "oracle", "precision": "fp64",
                   "sample": f"{nr} random query rows x all {n} reference windows ({dt:.1f} s, {how})"}
        line = {"metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
                "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True, "scaling": "strong",
                "vs_baseline": None, "dtype": {"fp64": "f64", "fp32": "f32"}.get(args.precision, args.precision),
                "data": "synthetic", "config": config_json(args, cfg), "roofline": roof, "cpu_baseline": cpu,
                "e2e": e2e, "gpu_launches": launches_per_step(args.precision, self_join) * args.steps,
                "clocks": clocks, "per_precision": per_prec, "context": context,
                "per_config_band": per_cfg or None, "computed_cells_per_s": cells * d / (ms * 1e-3),
                "stream": stream}
        if merge_check is not None:
            line["merge_check"] = merge_check
        if args.dry_run:
            line["dry_run"] = True
        print(json.dumps(line), flush=True)
    ctx.close()
    if world > 1:
        dist.destroy_process_group()
    return 0


if __name__ == "__main__":
    sys.exit(main())
