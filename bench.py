"""Benchmark of the mSTAMP hot path (BASELINE.json metric: d*n^2 matrix-profile cells*dims/s).

A "step" = one whole pass of the hot path (precompute -> fused diagonal kernel ->
finalize) over the workload, inputs resident in HBM.  Default workload: BASELINE
config C2 (self-join, d=16, n=65536, m=128, seeded random walk + planted motif), the
configuration the metric is quoted on, FP32 headline; every precision is also timed
and reported under "per_precision".

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
    """Algorithmic ALU-pipe ops per computed cell*dim: the d-way sort
    network (2 FMNMX per comparator, padded to a power of two) + 1 threshold compare per
    profile side updated (row; + column for the self-join)."""
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
    return ops / 2.0 if prec in ("fp16", "mixed", "fp16c") else ops


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
    Returns (cell*dims per second, rows, seconds, threads)."""
    import oracle
    oracle.build()
    T, Tr, m, e, n, d = cfg["T"], cfg["Tr"], cfg["m"], cfg["exclusion"], cfg["n"], cfg["d"]
    threads = os.cpu_count() or 1
    rng = np.random.default_rng(0)
    rows = np.sort(rng.choice(n, size=min(threads, n), replace=False))
    t0 = time.perf_counter()
    oracle.mstamp(T, m, e, Tr=Tr, rows=rows, nthreads=threads)
    dt = time.perf_counter() - t0
    for _ in range(2):  # calibrate (the first call also pays the O(n d m) window stats)
        nr = int(min(max_rows, max(len(rows), len(rows) * target_s / max(dt, 1e-6))))
        nr = max(threads, (nr // threads) * threads)
        rows = np.sort(rng.choice(n, size=min(nr, n), replace=False))
        t0 = time.perf_counter()
        oracle.mstamp(T, m, e, Tr=Tr, rows=rows, nthreads=threads)
        dt = time.perf_counter() - t0
        if dt > 0.5 * target_s or nr >= max_rows:
            break
    cells = len(rows) * n * d          # each sampled row: all n reference windows x d dims
    return cells / dt, len(rows), dt, threads


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
        v, nr, dt, th = oracle_sample(cfg, target_s=args.ref_seconds)
        vals.append(v)
        meta = (nr, dt, th)
    value = statistics.mean(vals)
    line = {"impl": "reference", "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": meta[1] * 1e3,
            "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "f64",
            "data": "synthetic", "config": config_json(args, cfg),
            "cpu_baseline": {"value": value, "unit": UNIT, "cores": meta[2], "kind": "oracle",
                             "sample": f"{meta[0]} random query rows x all n reference windows per step"},
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
def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--precision", default="fp32")
    ap.add_argument("--config", default="C2")
    ap.add_argument("--impl", default="native", choices=["native", "reference"])
    ap.add_argument("--ref-seconds", type=float, default=15.0)
    ap.add_argument("--no-per-precision", action="store_true")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-per-config", action="store_true",
                    help="skip the one-band throughput probes of the larger BASELINE configs")
    ap.add_argument("--backend", default="nccl", help="process-group backend for N>1 (gloo: functional "
                    "test of the multi-rank path, e.g. several ranks on one GPU via MP_BENCH_DEVICE)")
    args = ap.parse_args()
    args.warmup = max(args.warmup, 3)
    if args.impl == "reference":
        return run_reference(args)

    import torch
    import torch.distributed as dist
    from paper_conf_ipps_juryl022_b200 import mstamp

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("MP_BENCH_DEVICE", os.environ.get("LOCAL_RANK", "0")))
    torch.cuda.set_device(local)
    if world > 1:
        if args.backend == "nccl":
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
        else:
            dist.init_process_group(args.backend)
    dev = torch.device("cuda", local)
    cfg = datagen.make(args.config)
    d, n, m, e = cfg["d"], cfg["n"], cfg["m"], cfg["exclusion"]
    self_join = cfg["Tr"] is None
    T = torch.from_numpy(cfg["T"]).to(dev)
    Tr = None if self_join else torch.from_numpy(cfg["Tr"]).to(dev)
    ctx = mstamp.Context(local)
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)
    stream = torch.cuda.current_stream(dev)

    last = {}

    def one_step(prec):
        """One pass of the whole hot path; returns (device ms, main-kernel ms)."""
        P = torch.empty(d, n, dtype=torch.float64, device=dev)
        I = torch.empty(d, n, dtype=torch.int64, device=dev)
        last["P"], last["I"], last["prec"] = P, I, prec
        flush.fill_(1)
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        if world == 1:
            ctx.compute_device(T, m, P, I, prec, e, Tr=Tr, stream=stream)
        else:
            keys = torch.empty(mstamp.key_words(d, n, prec), dtype=torch.int64, device=dev)
            ctx.partial_device(T, m, keys, rank, world, prec, e, Tr=Tr, stream=stream)
            mstamp.merge_partials(ctx, keys, d, n, prec)
            if rank == 0:
                ctx.finalize_device(d, n, keys, P, I, prec, stream=stream)
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

    ms, kms, clocks = timed(args.precision, args.steps, args.warmup, sample_clocks=True)
    merge_check = None
    if world > 1 and rank == 0:
        # outside the timed region: the merged N-rank result must equal the 1-GPU result bit
        # for bit (fixed tile plan, lexicographic MINLOC merge: DESIGN.md section 10)
        P1 = torch.empty(d, n, dtype=torch.float64, device=dev)
        I1 = torch.empty(d, n, dtype=torch.int64, device=dev)
        ctx.compute_device(T, m, P1, I1, args.precision, e, Tr=Tr, stream=stream)
        torch.cuda.synchronize()
        merge_check = {"bit_identical_to_1gpu": bool(torch.equal(P1, last["P"]) and torch.equal(I1, last["I"]))}
        del P1, I1
    dn2 = d * n * n
    value = dn2 / (ms * 1e-3)

    per_prec = {}
    if not args.no_per_precision:
        for prec in ("fp64", "fp32", "mixed", "fp16"):
            if prec == args.precision:
                per_prec[prec] = {"value": value, "ms_per_step": ms, "main_kernel_ms": kms}
                continue
            p_ms, p_kms, _ = timed(prec, max(1, min(args.steps, 3)), 1)
            per_prec[prec] = {"value": dn2 / (p_ms * 1e-3), "ms_per_step": p_ms, "main_kernel_ms": p_kms}
        cells0 = computed_cells(n, e, self_join)
        for prec, v in per_prec.items():  # ALU roofline fraction of the main kernel per mode
            rate = cells0 * d / (v["main_kernel_ms"] * 1e-3)
            v["alu_frac"] = rate * alu_ops_mode(d, self_join, prec) / alu_peak_ops((clocks or {}).get("sm_mhz"))

    per_cfg = {}
    if not args.no_per_config and world == 1:
        for name, prec in (("C3", "fp32"), ("C3", "mixed"), ("C3", "fp16"), ("C4", "fp32"), ("C4", "mixed"),
                           ("C4", "fp64"), ("C5", "fp32"), ("C5", "mixed"), ("C5", "fp16"), ("C5", "fp64")):
            per_cfg[f"{name}/{prec}"] = band_probe(ctx, torch, dev, name, prec, peak=alu_peak_ops((clocks or {}).get("sm_mhz")))
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

    if rank == 0:
        peaks, src = load_peaks()
        cells = computed_cells(n, e, self_join)
        # roofline of the dominant kernel: algorithmic ops of the cells THIS launch computed (rank
        # 0's band when N > 1) over its CUDA-event duration
        band_cells = cells
        if world > 1:
            _, bc = mstamp.plan_bands(d, n, m, args.precision, e, self_join, world)
            band_cells = int(bc[0])
        ops = alu_ops_per_cell_dim(d, self_join) * band_cells * d
        lanes, lsrc = alu_lanes()
        run_mhz = (clocks or {}).get("sm_mhz") or NOMINAL_SM_MHZ
        peak_tops = alu_peak_ops(run_mhz) / 1e12
        achieved = ops / (kms * 1e-3) / 1e12 if kms > 0 else None
        roof = {"bound": "alu", "achieved": achieved, "peak": peak_tops, "unit": "Tops/s",
                "frac": achieved / peak_tops if achieved else None,
                "traffic": load_traffic(args.config, args.precision),
                "kernel": "mp_diag", "ops_per_cell_dim": alu_ops_per_cell_dim(d, self_join),
                "computed_cell_dims": band_cells * d,
                "peak_basis": f"{SM_COUNT} SM x {lanes:.2f} FMNMX lanes/SM/clk ({lsrc}: scripts/pipe_peaks.cu -> "
                              f"profiles/r1_pipe_peaks.json; MEASURED_PEAKS {src} has no ALU figure) x {run_mhz:.0f} MHz "
                              "(SM clock sampled during the timed region)"}
        cpu = None
        if not args.no_cpu_baseline and world == 1:
            v, nr, dt, th = oracle_sample(cfg, target_s=args.ref_seconds)
            cpu = {"value": v, "unit": UNIT, "cores": th, "kind": "oracle",
                   "sample": f"{nr} random query rows x all {n} reference windows ({dt:.1f} s)"}
        line = {"metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
                "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True, "scaling": "strong",
                "vs_baseline": None, "dtype": {"fp64": "f64", "fp32": "f32"}.get(args.precision, args.precision),
                "data": "synthetic", "config": config_json(args, cfg), "roofline": roof, "cpu_baseline": cpu,
                "e2e": e2e, "gpu_launches": launches_per_step(args.precision, self_join) * args.steps,
                "clocks": clocks, "per_precision": per_prec, "per_config_band": per_cfg or None,
                "computed_cells_per_s": cells * d / (ms * 1e-3)}
        if merge_check is not None:
            line["merge_check"] = merge_check
        print(json.dumps(line), flush=True)
    ctx.close()
    if world > 1:
        dist.destroy_process_group()
    return 0


if __name__ == "__main__":
    sys.exit(main())
