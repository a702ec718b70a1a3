#!/usr/bin/env python3
"""Benchmark: rerooted level-batched updatePartials on B200 (BASELINE.json metric).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config c1] [--precision 32]
                    [--impl ours|reference] [--no-secondary] [--no-strong]

A "step" is one pass of the whole hot path over the
workload: K1 transition matrices -> one updatePartials launch per level set
of the (re)rooted tree (K2; replayed from a CUDA graph) -> root integration K4
(-> NCCL all-reduce of the fp64 lnL sum when N > 1).  Rerooting + scheduling
(a1, a2) run once per tree on the host before the timed region, as in the
paper; the e2e leg repeats them every step.

`value` = effective GFLOPS of Eq. (1) (flops per pattern per pass
(n-1) c s (4s-1), A16) summed over ranks / max-over-ranks device
time of the K steps.  Inputs are resident in HBM; L2 (126 MB) is flushed by a
512 MiB memset before every step, outside the per-step CUDA events.  The K
steps are timed with the library's profiling off; a second pass of K steps
with it on (CUDA events around every graph replay of the updatePartials
region) gives the region's duration for `updatePartials` and `roofline`.

Multi-GPU (one process per GPU; `--gpus N` without torchrun re-launches itself
under torch.distributed.run): the headline is weak scaling -- every rank owns
its own 10,000-pattern slice (patterns are independent) -- and
`strong_scaling` rides along: configs[4] (4,096-tip pectinate, 4,194,304
patterns) split over the N ranks through ShardedTreeLikelihood; the only
collective is the all-reduce of the per-rank lnL.

Ride-alongs (rank 0 prints one JSON line): `reroot` (original-root and
sequential schedules of the same workload), `hbm_regime` (configs[2]),
`codon` (configs[3], tcgen05), `reroot_target` (1,024-tip pectinate at
512/2,048/4,096 patterns, interleaved arms, best and median over 200 reps,
identical-schedule control), `stored_factors` (the paper's rescale-frequency
regime), `strong_scaling`, `cpu_baseline` (the oracle on 1 core
and on all cores).
"""
from __future__ import annotations

import argparse
import json
import math
import os
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

from workloads import CONFIGS, config_workload, make_workload  # noqa: E402

CONFIG_DESC = {
    "c0_hky": "configs[0]: 8-tip pectinate, HKY, 1 category, 1,000 patterns",
    "c1": "configs[1]: 128-tip pectinate rerooted vs original, GTR+G4, 10,000 patterns per GPU",
    "c2": "configs[2]: 1,024-tip Yule rerooted, GTR+G4, 100,000 patterns per GPU",
    "c2_paper": "1,024-tip paper-random (PAPER.md:148) rerooted, GTR+G4, 100,000 patterns per GPU",
    "c3": "configs[3]: 256-tip paper-random rerooted, GY94+G4 (61 states), 10,000 patterns per GPU",
    "c4": "configs[4]: 4,096-tip pectinate rerooted, GTR+G4, 4,194,304 patterns (strong scaling)",
}
METRIC = "updatePartials GFLOPS rerooted vs original root; %HBM roofline; 1/2/4/8 GPU"
TF32_PEAK_NOTE = "tf32 dense = bf16 measured burst x 1/2 (B200 nominal 1.1 vs 2.25 PFLOP/s)"


def flops_per_pass(n, p, c, s):
    return (n - 1) * p * c * s * (4 * s - 1)


def bytes_per_pass(ops, n, p, c, s, elt, cumulative=True):
    """Algorithmic HBM bytes of all updatePartials launches of one pass
    (DESIGN.md §6): per op and pattern, each internal child's c*s*elt
    partials (+4 B cumulative exponent), each tip child's 1 B state, the
    c*s*elt output and the 4 B exponent."""
    per = 0
    for o in ops:
        for ch in (int(o["child1"]), int(o["child2"])):
            per += 1 if ch < n else c * s * elt + (4 if cumulative else 0)
        per += c * s * elt + 4
    return per * p


def internal_children(ops, n):
    return sum(int(int(o["child1"]) >= n) + int(int(o["child2"]) >= n) for o in ops)


def cpu_info():
    model = "unknown"
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                model = line.split(":", 1)[1].strip()
                break
    except OSError:
        pass
    return {"cores": len(os.sched_getaffinity(0)), "model": model}


# ----------------------------------------------------------------------------- clocks
class ClockSampler:
    """SM clocks and throttle reasons during the timed region: NVML polled every
    5 ms from a thread (plus `sample()` calls the timing loop makes while the
    GPU is still busy with enqueued steps, so even a short region is covered);
    nvidia-smi -lms 100 when NVML is unavailable."""
    FIELDS = ("clocks.sm,clocks.max.sm,clocks_event_reasons.hw_slowdown,"
              "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
              "clocks_event_reasons.sw_power_cap")
    NAMES = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]

    def __init__(self, device: int):
        self.rows, self.proc, self.nv, self.t = [], None, None, None
        self._stop = threading.Event()
        try:
            import pynvml as nv
            nv.nvmlInit()
            self.h = nv.nvmlDeviceGetHandleByIndex(device)
            self.nv = nv
            self.bits = [nv.nvmlClocksEventReasonHwSlowdown, nv.nvmlClocksEventReasonHwThermalSlowdown,
                         nv.nvmlClocksEventReasonSwThermalSlowdown, nv.nvmlClocksEventReasonSwPowerCap]
            self.max_mhz = float(nv.nvmlDeviceGetMaxClockInfo(self.h, nv.NVML_CLOCK_SM))
            self.t = threading.Thread(target=self._poll, daemon=True)
            self.t.start()
            return
        except Exception:
            self.nv = None
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", f"--query-gpu={self.FIELDS}", "--format=csv,noheader,nounits",
                 "-i", str(device), "-lms", "100"], stdout=subprocess.PIPE,
                stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception:
            self.proc = None

    def sample(self):
        if self.nv is None:
            return
        try:
            sm = float(self.nv.nvmlDeviceGetClockInfo(self.h, self.nv.NVML_CLOCK_SM))
            r = self.nv.nvmlDeviceGetCurrentClocksEventReasons(self.h)
            self.rows.append((sm, self.max_mhz, [bool(r & b) for b in self.bits]))
        except Exception:
            pass

    def _poll(self):
        while not self._stop.wait(0.005):
            self.sample()

    def _read(self):
        for line in self.proc.stdout:
            parts = [x.strip() for x in line.strip().split(",")]
            if len(parts) != 6:
                continue
            try:
                self.rows.append((float(parts[0]), float(parts[1]), [v.lower() == "active" for v in parts[2:]]))
            except ValueError:
                continue

    def stop(self) -> dict:
        if self.nv is None and self.proc is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        self._stop.set()
        if self.proc is not None:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=5)
            except Exception:
                self.proc.kill()
        if self.t is not None:
            self.t.join(timeout=2)
        rows = list(self.rows)
        sm = [r[0] for r in rows]
        reasons = sorted({nm for r in rows for nm, on in zip(self.NAMES, r[2]) if on})
        return {"sm_mhz": float(np.median(sm)) if sm else None,
                "sm_max_mhz": float(max(r[1] for r in rows)) if rows else None,
                "reasons": reasons, "samples": len(sm),
                "source": "nvml" if self.nv is not None else "nvidia-smi"}


# ----------------------------------------------------------------------------- workloads
def rank_workload(cfg: str, rank: int, world: int, seed: int = 1):
    """Weak scaling (c0-c3): each rank owns patterns [r p, (r+1) p) of a global
    alignment of world*p patterns.  c4 is strong scaling (see c4_slice)."""
    base = dict(CONFIGS[cfg])
    p = base["p"]
    if cfg == "c4":
        w = config_workload(cfg, seed=seed, p=1)
        lo, hi = pattern_slice_of(p, rank, world)
        w.tips = c4_tips(w.n, lo, hi, seed)
        w.pattern_weights = np.ones(hi - lo)
        return w, "strong"
    w = config_workload(cfg, seed=seed, p=p * world)
    w.tips = np.ascontiguousarray(w.tips[:, rank * p:(rank + 1) * p])
    w.pattern_weights = np.ones(p)
    return w, "weak"


def pattern_slice_of(p, rank, world):
    chunk = math.ceil(p / world)
    lo = min(p, rank * chunk)
    return lo, min(p, lo + chunk)


C4_BLOCK = 1 << 16


def c4_tips(n, lo, hi, seed=1):
    """Uniform tip states of configs[4]'s global alignment, generated in fixed
    blocks of 65,536 patterns (block b seeded by (seed, 7919, b)), so every
    rank count N sees the same global alignment."""
    out = np.empty((n, hi - lo), dtype=np.uint8)
    b0, b1 = lo // C4_BLOCK, (hi + C4_BLOCK - 1) // C4_BLOCK
    for b in range(b0, b1):
        rng = np.random.default_rng(np.random.SeedSequence([seed, 7919, b]))
        blk = rng.integers(0, 4, size=(n, C4_BLOCK), dtype=np.uint8)
        a, z = max(lo, b * C4_BLOCK), min(hi, (b + 1) * C4_BLOCK)
        out[:, a - lo:z - lo] = blk[:, a - b * C4_BLOCK:z - b * C4_BLOCK]
    return out


def ncu_traffic(key: str):
    """DRAM bytes per updatePartials launch from the committed ncu capture
    (profiles/ncu_traffic.json); null when there is none for this config."""
    try:
        return json.load(open(os.path.join(ROOT, "profiles", "ncu_traffic.json"))).get(key)
    except Exception:
        return None


def measured_peaks():
    try:
        return json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json"))), "measured"
    except Exception:
        return {"hbm_gbs": 6650.0, "bf16_tflops": 2250.0}, "fallback (B200_PROFILING.md)"


# ----------------------------------------------------------------------------- oracle timing
MAX_ORACLE_PROCS = 64


def _oracle_shard(args):
    """One worker of the oracle timing (1 BLAS thread per process): builds its
    contiguous pattern shard of configs[cfg] (untimed), then times `reps`
    plain prunes of it.  Returns the per-rep seconds."""
    from threadpoolctl import threadpool_limits

    from oracle import model as om, pruning
    cfg, lo, hi, reps = args
    w = config_workload(cfg, seed=1, p=hi)
    tips = np.ascontiguousarray(w.tips[:, lo:hi])
    Q = om.rate_matrix(w.model)
    out = []
    with threadpool_limits(limits=1):
        for _ in range(reps):
            t0 = time.perf_counter()
            pruning.prune(w.tree, Q, w.model.pi, w.rates, w.cat_weights, tips, np.ones(hi - lo))
            out.append(time.perf_counter() - t0)
    return out


def oracle_pool_times(cfg, per_core, procs, reps):
    """`procs` processes (spawned, one per core), each pruning its own shard of
    per_core patterns `reps` times concurrently; per rep, the slowest worker's
    time (all shards done)."""
    import multiprocessing as mproc
    jobs = [(cfg, k * per_core, (k + 1) * per_core, reps) for k in range(procs)]
    with mproc.get_context("spawn").Pool(procs) as pool:
        res = pool.map(_oracle_shard, jobs)
    return [max(r[i] for r in res) for i in range(reps)]


def oracle_rate(cfg: str, budget_s: float, cores: int):
    """The oracle as it stands (never tuned), fp64 NumPy/SciPy, on a bounded
    pattern sample of configs[cfg]: (GFLOPS on 1 core, GFLOPS on min(cores,
    64) concurrent processes over contiguous pattern shards, procs, sample)."""
    w = config_workload(cfg, seed=1, p=min(CONFIGS[cfg]["p"], 64))
    t1 = _oracle_shard((cfg, 0, 64, 1))[0]
    per_core = int(max(16, min(4096, CONFIGS[cfg]["p"] // max(1, min(cores, MAX_ORACLE_PROCS)),
                               64 * budget_s / 2 / max(t1, 1e-3))))
    one = _oracle_shard((cfg, 0, per_core, 1))[0]
    fl = flops_per_pass(w.n, per_core, w.c, w.s)
    v1 = fl / one / 1e9
    procs = min(cores, MAX_ORACLE_PROCS)
    vall = None
    if procs > 1:
        t = oracle_pool_times(cfg, per_core, procs, 1)[0]
        vall = fl * procs / t / 1e9
    return v1, vall, procs, (f"{per_core} patterns per core x full {w.n}-tip tree of {cfg}, one pass "
                             f"({one:.1f} s on 1 core)")


# ----------------------------------------------------------------------------- reference arm
def run_reference(args, rank, world):
    """--impl reference: the fp64 oracle (test infrastructure) timed as it
    stands on the host cores (one process per core over contiguous pattern
    shards), each step a bounded pattern sample of the workload."""
    if rank != 0:
        return
    info = cpu_info()
    cores = min(info["cores"], MAX_ORACLE_PROCS)
    cfg = args.config
    w = config_workload(cfg, seed=1, p=64)
    t1 = _oracle_shard((cfg, 0, 64, 1))[0]
    per_step_budget = 120.0 / (args.steps + args.warmup)
    per_core = int(max(16, min(4096, CONFIGS[cfg]["p"] // cores, 64 * per_step_budget / max(t1, 1e-3))))
    times = oracle_pool_times(cfg, per_core, cores, args.warmup + args.steps)
    dt = sum(times[args.warmup:])
    sample = per_core * cores
    val = flops_per_pass(w.n, sample, w.c, w.s) * args.steps / dt / 1e9
    line = {
        "impl": "reference", "metric": METRIC, "value": val, "unit": "GFLOPS",
        "n_gpus": world, "steps": args.steps, "warmup": args.warmup,
        "ms_per_step": dt / args.steps * 1e3, "higher_is_better": True, "scaling": "weak",
        "vs_baseline": None, "dtype": "f64", "data": "synthetic (seeded, workloads/)",
        "config": {"workload": CONFIG_DESC.get(cfg, cfg), "sample_patterns": sample,
                   "schedule": "post-order (oracle)"},
        "cpu_baseline": {"value": val, "unit": "GFLOPS", "cores": cores, "kind": "oracle",
                         "cpu_model": info["model"], "host_cores": info["cores"],
                         "sample": f"{sample} patterns ({per_core} per core, one process per core) of "
                                   f"{CONFIGS[cfg]['p']}, full {w.n}-tip tree, per step"},
        "e2e": {"value": val, "unit": "GFLOPS", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)


# ----------------------------------------------------------------------------- our arm
def relaunch_under_torchrun(args) -> int:
    """`bench.py --gpus N` started without torchrun: one process per GPU."""
    import socket
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
           "--master-addr", "127.0.0.1", "--master-port", str(port), os.path.abspath(__file__)] + sys.argv[1:]
    return subprocess.call(cmd)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=200)
    ap.add_argument("--warmup", type=int, default=10)
    ap.add_argument("--config", default="c1", choices=sorted(CONFIG_DESC))
    ap.add_argument("--precision", type=int, default=32, choices=(32, 64))
    ap.add_argument("--impl", default="ours", choices=("ours", "reference"))
    ap.add_argument("--no-graph", action="store_true")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-secondary", action="store_true",
                    help="skip the ride-along measurements (hbm_regime, codon, reroot_target, stored_factors)")
    ap.add_argument("--no-strong", action="store_true", help="skip the configs[4] strong-scaling object")
    ap.add_argument("--reps", type=int, default=200, help="reps per arm of reroot_target")
    args = ap.parse_args()
    args.warmup = max(args.warmup, 3)

    if args.gpus > 1 and "WORLD_SIZE" not in os.environ:
        sys.exit(relaunch_under_torchrun(args))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))

    if args.impl == "reference":
        run_reference(args, rank, world)
        return

    import torch
    if not torch.cuda.is_available():
        raise SystemExit("bench.py needs a CUDA device (no CPU fallback)")
    local = local % torch.cuda.device_count()  # (several ranks may share a GPU in wiring tests)
    torch.cuda.set_device(local)
    torch.cuda.set_stream(torch.cuda.Stream())  # capturable, non-legacy stream for everything timed
    dist = None
    backend = os.environ.get("RRL_DIST_BACKEND", "nccl")  # gloo: CPU-side test of the wiring
    if world > 1:
        import torch.distributed as dist
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
        else:
            dist.init_process_group(backend)

    from paper_conf_ipps_ayresc18_b200 import build as _b
    _b.build()
    from paper_conf_ipps_ayresc18_b200 import TreeLikelihood, rrl as R
    from paper_conf_ipps_ayresc18_b200.parallel import ShardedTreeLikelihood, allreduce_sum_

    stream = torch.cuda.current_stream()
    flush = torch.empty(512 * 1024 * 1024 // 4, dtype=torch.float32, device="cuda")
    d_out = torch.zeros(1, dtype=torch.float64, device="cuda")
    peaks, peak_src = measured_peaks()
    hbm = float(peaks.get("hbm_gbs", 6650.0))
    tf32_peak = float(peaks.get("bf16_tflops", 2250.0)) / 2
    fp64_peak = 148 * 64 * 2 * 1.965e9 / 1e12
    info = cpu_info()

    def maxall(x):
        if dist is None:
            return x
        t = torch.tensor([x], dtype=torch.float64, device="cuda")
        if backend == "nccl":
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
        else:
            h = t.cpu()
            dist.all_reduce(h, op=dist.ReduceOp.MAX)
            t.copy_(h)
        return float(t.item())

    def barrier():
        torch.cuda.synchronize()
        if dist is not None:
            dist.barrier()
        torch.cuda.synchronize()

    def make(w, mode, precision, reuse=False, fused=False):
        nbuf = None
        if reuse:
            nbuf = R.rrl_reroot_and_schedule(w.n, w.tree.parent, w.tree.blen, mode, True)["buffer_count"]
        tl = TreeLikelihood(w.n, w.p, w.s, w.c, precision=precision, device=local,
                            cuda_graph=not args.no_graph, buffer_count=nbuf,
                            stream_ptr=stream.cuda_stream, fused_pass=fused)
        tl.set_model_params(w.model, w.rates, w.cat_weights)
        tl.set_tips(w.tips)
        tl.set_pattern_weights(w.pattern_weights)
        tl.set_tree(w.tree.parent, w.tree.blen, mode, reuse_buffers=reuse)
        return tl

    def step(tl):
        tl.update()
        tl.root_loglik_device(d_out.data_ptr())
        if dist is not None:
            allreduce_sum_(d_out)

    def timed(tl, steps, warmup, clocks=None, fn=None):
        """Per-step CUDA events on the launching stream; L2 flushed before
        every step outside the events; barrier + synchronize on both sides.
        Two passes of `steps` steps: the step times come from a pass with the
        library's profiling off (its event records between launches would sit
        inside the timed step); the updatePartials region times (the
        roofline's launch durations) from a second pass with it on."""
        fn = fn or step
        for _ in range(warmup):
            flush.zero_()
            fn(tl)
        barrier()

        def run(profile):
            evs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True))
                   for _ in range(steps)]
            if profile:  # CUDA events on this stream around every graph replay of the region
                R.rrl_set_profiling(tl.inst, True)
                R.rrl_reset_profile(tl.inst)
            for i, (a, b) in enumerate(evs):
                flush.zero_()
                a.record(stream)
                fn(tl)
                b.record(stream)
                if clocks is not None and not profile and i % 16 == 15:
                    clocks.sample()  # the GPU is still running enqueued steps
            if clocks is not None and not profile:
                clocks.sample()
            barrier()
            per = [a.elapsed_time(b) for a, b in evs]
            prof = None
            if profile:
                prof = R.rrl_get_profile(tl.inst)
                R.rrl_set_profiling(tl.inst, False)
            return per, prof

        per, _ = run(False)
        _, prof = run(True)
        return maxall(sum(per)), prof, {"best": maxall(min(per)), "median": maxall(float(np.median(per)))}

    def roofline_of(cfg, precision, w, sched, part_ms, launches_per_pass):
        n, p, c, s = w.n, w.p, w.c, w.s
        elt = 4 if precision == 32 else 8
        bpp = bytes_per_pass(sched["ops"], n, p, c, s, elt)
        achieved = bpp / (part_ms * 1e-3) / 1e9
        rf = {"bound": "hbm", "achieved": achieved, "peak": hbm, "unit": "GB/s", "frac": achieved / hbm,
              "traffic": ncu_traffic(f"{cfg}_fp{precision}"),
              "kernel": "k_partials_nuc / k_partials_nuc_bulk (updatePartials, one launch per level set)",
              "algorithmic_bytes_per_pass": bpp, "algorithmic_bytes_per_launch": bpp / max(1.0, launches_per_pass),
              "launches_per_pass": launches_per_pass,
              "peak_source": f"{peak_src} hbm_gbs (MEASURED_PEAKS.json)",
              "timing": "CUDA events on the launching stream around every CUDA-graph replay of the "
                        "updatePartials region inside the timed steps; per-launch duration = region time / "
                        "level-set launches"}
        if s == 61:
            # contractions the kernels execute: internal children only (a tip child
            # is a gather of P's column); 3xTF32 = 3 MMAs on the 64-padded operands
            ic = internal_children(sched["ops"], n)
            eff = flops_per_pass(n, p, c, s) / (part_ms * 1e-3) / 1e12
            if precision == 32:
                mma = ic * p * c * 3 * 2 * 64 * 64
                rf.update({"kernel": "k_partials_codon_tc5 (TMA-fed tcgen05 kind::tf32, 3xTF32)",
                           "tensor": {"executed_tflops": mma / (part_ms * 1e-3) / 1e12, "peak_tflops": tf32_peak,
                                      "frac": mma / (part_ms * 1e-3) / 1e12 / tf32_peak,
                                      "peak_source": TF32_PEAK_NOTE,
                                      "counted": f"{ic} internal-child contractions x p x c x 3 MMAs x "
                                                 "2 x 64 x 64 (tip children are P-column gathers)"},
                           "effective_tflops": eff})
            else:
                ex = ic * p * c * 2 * s * s + (n - 1) * p * c * s
                ach = ex / (part_ms * 1e-3) / 1e12
                rf.update({"bound": "alu", "achieved": ach, "peak": fp64_peak, "unit": "TFLOP/s",
                           "frac": ach / fp64_peak, "hbm_achieved_gbs": achieved,
                           "kernel": "k_partials_codon (SIMT fp64)",
                           "peak_source": "derived: 148 SMs x 64 FP64 lanes x 2 flop x 1.965 GHz",
                           "flops": f"executed: {ic} internal-child mat-vecs x 2 s^2 + the s-wide "
                                    "products, per pattern and category (tip children are gathers)",
                           "effective_tflops": eff})
        return rf

    def measure(cfg, precision, steps, warmup, arms=("level", "sequential")):
        w, scaling = rank_workload(cfg, rank, world)
        n, p, c, s = w.n, w.p, w.c, w.s
        reuse = cfg == "c4"  # 4,096 x 4 M patterns: liveness buffer reuse (1.1 TB otherwise)
        if reuse:
            arms = ()
        tl = make(w, "reroot", precision, reuse)
        sched = tl.sched
        clocks = ClockSampler(local)
        ms, prof, bm = timed(tl, steps, warmup, clocks)
        clk = clocks.stop()
        fl = flops_per_pass(n, p, c, s)
        part_ms = maxall(prof["partials_ms"]) / steps
        lpp = prof["partials_launches"] / steps
        res = {
            "cfg": cfg, "w": w, "tl": tl, "scaling": scaling, "n": n, "p": p, "c": c, "s": s,
            "value": fl * world * steps / (ms * 1e-3) / 1e9, "ms_per_step": ms / steps,
            "ms_per_step_best": bm["best"], "ms_per_step_median": bm["median"],
            "launches": prof["kernel_launches"], "clocks": clk, "sets": sched["set_count"], "fl": fl,
            "updatePartials": {"ms_per_pass": part_ms, "launches_per_pass": lpp,
                               "gflops": fl / (part_ms * 1e-3) / 1e9,
                               "pattern_node_updates_per_s": (n - 1) * p / (part_ms * 1e-3),
                               "share_of_step": part_ms / (ms / steps)},
            "roofline": roofline_of(cfg, precision, w, sched, part_ms, lpp),
            "lnL": float(d_out.item()),
        }
        other = {}
        for mode in arms:
            to = make(w, mode, precision)
            ms_o, prof_o, _ = timed(to, steps, warmup)
            other[mode] = (ms_o, maxall(prof_o["partials_ms"]) / steps, to.sched["set_count"])
            to.close()
        if "level" in other:
            ms_o, po, so = other["level"]
            res["reroot"] = {
                "sets": sched["set_count"], "sets_original": so,
                "theoretical_speedup": so / sched["set_count"],
                "step_speedup": ms_o / ms, "updatePartials_speedup": po / part_ms,
                "original_gflops": fl * world * steps / (ms_o * 1e-3) / 1e9,
                "original_updatePartials_ms": po,
                "paper_context": "BEAGLE CUDA on Quadro GP100: up to 1.93x (pectinate, 406 OTUs, "
                                 "512 patterns, PAPER.md:258); mean 1.26x (random 256 OTUs, PAPER.md:230)"}
            if "sequential" in other:
                _, ps, ss = other["sequential"]
                # S_conc = T_sequential / T_level (Table III, reading A18)
                res["reroot"]["S_conc"] = {"original": ps / po, "rerooted": ps / part_ms,
                                           "theory_original": ss / so, "theory_rerooted": ss / sched["set_count"],
                                           "sequential_updatePartials_ms": ps}
        return res

    # ---------------- headline
    prim = measure(args.config, args.precision, args.steps, args.warmup)
    w, tl = prim["w"], prim["tl"]
    n, p = prim["n"], prim["p"]

    # ---------------- e2e through the public API with host buffers (pinned), every step:
    # reroot + schedule, H2D tips + branch lengths, pass, D2H of the lnL.
    reuse = args.config == "c4"
    pinned = torch.empty(w.tips.shape, dtype=torch.uint8, pin_memory=True).numpy()
    pinned[:] = w.tips
    e2e_steps = max(3, min(args.steps, 50))
    for _ in range(2):
        tl.set_tips(pinned)
        tl.set_tree(w.tree.parent, w.tree.blen, "reroot", reuse_buffers=reuse)
        tl.loglik()
    barrier()
    t0 = time.perf_counter()
    for _ in range(e2e_steps):
        tl.set_tips(pinned)
        tl.set_tree(w.tree.parent, w.tree.blen, "reroot", reuse_buffers=reuse)
        tl.update()
        tl.root_loglik_device(d_out.data_ptr())
        if dist is not None:
            allreduce_sum_(d_out)
        float(d_out.item())
    e2e_s = maxall(time.perf_counter() - t0)
    e2e_val = prim["fl"] * world * e2e_steps / e2e_s / 1e9
    # bytes copied per step: the tip states (set_tips); the branch lengths and
    # matrix indices are unchanged step to step, so K1 reuses their device copy
    h2d = int(w.tips.nbytes)

    # ---------------- stored factors (the paper's timed regime: new factors once
    # per 1,000 reps; reading A6): ops apply the exponents the
    # write pass stored (dest_scale_read) instead of computing new ones
    stored = None
    if not args.no_secondary and prim["s"] == 4 and not reuse:
        tn = TreeLikelihood(w.n, w.p, w.s, w.c, precision=args.precision, device=local,
                            cumulative_scaling=False, cuda_graph=not args.no_graph, stream_ptr=stream.cuda_stream)
        tn.set_model_params(w.model, w.rates, w.cat_weights)
        tn.set_tips(w.tips)
        tn.set_tree(w.tree.parent, w.tree.blen, "reroot")
        tn.update()
        ops_r = tn.ops.copy()
        ops_r["dest_scale_read"] = ops_r["dest_scale_write"]
        ops_r["dest_scale_write"] = -1

        def step_read(t):
            R.rrl_update_transition_matrices(t.inst, 0, t.matrix_idx, t.t)
            R.rrl_update_partials(t.inst, ops_r, t.offsets)
            R.rrl_calculate_root_log_likelihoods_device(t.inst, t.root_buffer, 0, 0, t.n_scale - 1,
                                                        d_out.data_ptr())
            if dist is not None:
                allreduce_sum_(d_out)
        ms_r, prof_r, _ = timed(tn, args.steps, args.warmup, fn=step_read)
        pr = maxall(prof_r["partials_ms"]) / args.steps
        stored = {"value": prim["fl"] * world * args.steps / (ms_r * 1e-3) / 1e9, "unit": "GFLOPS",
                  "ms_per_step": ms_r / args.steps, "updatePartials_ms_per_pass": pr,
                  "vs_write_every_pass": prim["updatePartials"]["ms_per_pass"] / pr,
                  "mode": "per-node exponents stored by one write pass, applied by every timed pass "
                          "(dest_scale_read), as with --rescale-frequency 1000 (PAPER.md:180)"}
        tn.close()
    tl.close()

    # ---------------- the HBM-bound regime (configs[2]) beside the launch-bound headline
    sec = codon = None
    if args.config == "c1" and not args.no_secondary:
        r2 = measure("c2", args.precision, min(args.steps, 30), args.warmup, arms=("level",))
        r2["tl"].close()
        sec = r2
        r3 = measure("c3", 32, min(args.steps, 30), args.warmup, arms=("level",))
        r3["tl"].close()
        codon = r3

    # ---------------- reroot speedup target (north star: >= 1.8x on 1,024-tip
    # pectinate trees): interleaved arms, best and median, identical-schedule control
    target = None
    if not args.no_secondary:
        target = {"workload": "1,024-tip pectinate, GTR+G4, fp32, rescaling every pass, L2 flushed before "
                              "every rep", "reps": args.reps, "points": []}
        for pp in (512, 2048, 4096):
            wt = make_workload(tree_kind="pectinate", n=1024, p=pp, model="gtr", c=4, seed=1)
            arms = {"original": make(wt, "level", 32), "rerooted": make(wt, "reroot", 32),
                    "control": make(wt, "level", 32)}
            for a in arms.values():
                for _ in range(3):
                    a.update()
                R.rrl_set_profiling(a.inst, True)
            times = {k: [] for k in arms}
            barrier()
            for _ in range(args.reps):
                for k, a in arms.items():       # interleaved: drifts hit every arm alike
                    flush.zero_()
                    R.rrl_reset_profile(a.inst)
                    a.update()
                    times[k].append(R.rrl_get_profile(a.inst)["partials_ms"])
            st = {k: {"best_ms": maxall(min(v)), "median_ms": maxall(float(np.median(v)))}
                  for k, v in times.items()}
            bound = arms["original"].sched["set_count"] / arms["rerooted"].sched["set_count"]
            target["points"].append({
                "patterns": pp, "sets": [arms["original"].sched["set_count"], arms["rerooted"].sched["set_count"]],
                "bound": bound, "arms": st,
                "speedup_best": st["original"]["best_ms"] / st["rerooted"]["best_ms"],
                "speedup_median": st["original"]["median_ms"] / st["rerooted"]["median_ms"],
                "control_ratio_median": st["original"]["median_ms"] / st["control"]["median_ms"],
                "rerooted_gflops_median": flops_per_pass(1024, pp, 4, 4) / (st["rerooted"]["median_ms"] * 1e-3) / 1e9})
            for a in arms.values():
                a.close()
        target["met_1.8x_median"] = all(pt["speedup_median"] >= 1.8 for pt in target["points"])
        target["control_within_2pct"] = all(abs(pt["control_ratio_median"] - 1) <= 0.02 for pt in target["points"])

    # ---------------- strong scaling: configs[4] split over the N ranks (ShardedTreeLikelihood)
    strong = None
    if not args.no_strong and args.config != "c4":
        P4 = CONFIGS["c4"]["p"]
        w4 = config_workload("c4", seed=1, p=1)
        lo, hi = pattern_slice_of(P4, rank, world)
        nb = R.rrl_reroot_and_schedule(w4.n, w4.tree.parent, w4.tree.blen, "reroot", True)["buffer_count"]
        sh = ShardedTreeLikelihood(w4.n, P4, 4, 4, rank, world, precision=32, device=local,
                                   stream_ptr=stream.cuda_stream, buffer_count=nb)
        sh.set_model_params(w4.model, w4.rates, w4.cat_weights)
        sh.set_tips_local(c4_tips(w4.n, lo, hi))
        sh.set_pattern_weights(np.ones(P4))
        sh.set_tree(w4.tree.parent, w4.tree.blen, "reroot", reuse_buffers=True)
        k4, w4u = 5, 3
        ms4, prof4, bm4 = timed(sh.tl, k4, w4u, fn=lambda t: sh.loglik_device())
        p4 = maxall(prof4["partials_ms"]) / k4
        fl4 = flops_per_pass(w4.n, P4, 4, 4)
        strong = {"workload": CONFIG_DESC["c4"], "n_gpus": world, "patterns_total": P4,
                  "patterns_per_rank": hi - lo, "buffers_per_rank": nb,
                  "value": fl4 * k4 / (ms4 * 1e-3) / 1e9, "unit": "GFLOPS", "ms_per_step": ms4 / k4,
                  "ms_per_step_best": bm4["best"], "updatePartials_ms_per_pass": p4,
                  "roofline_frac_per_rank": bytes_per_pass(sh.tl.sched["ops"], w4.n, hi - lo, 4, 4, 4)
                  / (p4 * 1e-3) / 1e9 / hbm,
                  "lnL": float(sh.d_out.item()), "path": "ShardedTreeLikelihood: pattern slice per rank, "
                  "K1 + 2,048 level-set launches + K4 + all-reduce of the fp64 lnL"}
        sh.close()

    if rank != 0:
        if dist is not None:
            dist.destroy_process_group()
        return
    cpu = None
    if not args.no_cpu_baseline:
        v1, vall, procs, smp = oracle_rate(args.config, 12.0, info["cores"])
        cpu = {"value": vall if vall is not None else v1, "unit": "GFLOPS", "cores": procs,
               "host_cores": info["cores"], "kind": "oracle", "cpu_model": info["model"], "value_1core": v1,
               "value_all_cores": vall,
               "sample": smp + f"; all-cores value = {procs} concurrent processes (one per core, 1 BLAS "
                               "thread each) over contiguous pattern shards, slowest shard's time"}
    out = {
        "metric": METRIC,
        "value": prim["value"],
        "unit": "GFLOPS",
        "n_gpus": world,
        "steps": args.steps,
        "warmup": args.warmup,
        "ms_per_step": prim["ms_per_step"],
        "ms_per_step_best": prim["ms_per_step_best"],
        "ms_per_step_median": prim["ms_per_step_median"],
        "higher_is_better": True,
        "scaling": prim["scaling"],
        "vs_baseline": None,
        "dtype": f"f{args.precision}",
        "data": "synthetic (seeded workloads/: tree, GTR+G4 parameters, uniform alignment)",
        "config": {"workload": CONFIG_DESC[args.config], "n_tips": n, "patterns_per_gpu": p,
                   "categories": prim["c"], "states": prim["s"], "schedule": "reroot",
                   "sets": prim["sets"], "cuda_graph": not args.no_graph,
                   "l2": "flushed before every step (512 MiB memset, outside the step events)"},
        "reroot": prim.get("reroot"),
        "updatePartials": prim["updatePartials"],
        "roofline": prim["roofline"],
        "cpu_baseline": cpu,
        "e2e": {"value": e2e_val, "unit": "GFLOPS", "h2d_bytes_per_step": h2d,
                "d2h_bytes_per_step": 8, "steps": e2e_steps,
                "path": "TreeLikelihood: set_tips (pinned H2D of every tip row) + rrl_reroot_and_schedule + "
                        "K1 + level-set K2 + K4 + D2H lnL"},
        "gpu_launches": int(prim["launches"]),
        "clocks": prim["clocks"],
        "lnL": prim["lnL"],
    }
    if stored is not None:
        out["stored_factors"] = stored
    for key, r in (("hbm_regime", sec), ("codon", codon)):
        if r is not None:
            out[key] = {"workload": CONFIG_DESC[r["cfg"]], "value": r["value"], "unit": "GFLOPS",
                        "ms_per_step": r["ms_per_step"], "ms_per_step_median": r["ms_per_step_median"],
                        "reroot": r.get("reroot"), "updatePartials": r["updatePartials"],
                        "roofline": r["roofline"], "gpu_launches": int(r["launches"]), "clocks": r["clocks"]}
    if target is not None:
        out["reroot_target"] = target
    if strong is not None:
        out["strong_scaling"] = strong
    print(json.dumps(out), flush=True)
    if dist is not None:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
