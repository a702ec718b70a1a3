#!/usr/bin/env python3
"""Benchmark: rerooted level-batched updatePartials on B200 (BASELINE.json metric).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config c1] [--precision 32]
                    [--impl ours|reference]

A "step" is one pass of the whole hot path over the
workload: K1 transition matrices -> one updatePartials launch per level set
of the (re)rooted tree (K2; replayed from a CUDA graph) -> root integration K4
(-> NCCL all-reduce of the fp64 lnL sum when N > 1).  Rerooting + scheduling
(a1, a2) run once per tree on the host before the timed region, as in the
paper; the e2e leg repeats them every step.

`value` = effective GFLOPS of Eq. (1) (flops per pattern per pass
(n-1) c s (4s-1), A16) summed over ranks / max-over-ranks device
time of the K steps.  Inputs are resident in HBM; L2 (126 MB) is flushed by a
512 MiB memset before every step, outside the per-step CUDA events.

Multi-GPU: weak scaling -- every rank owns its own 10,000-pattern slice
(patterns are independent) of a global alignment of N x p
patterns; the only collective is the all-reduce of the per-rank lnL.
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

from workloads import CONFIGS, config_workload  # noqa: E402

CONFIG_DESC = {
    "c0_hky": "configs[0]: 8-tip pectinate, HKY, 1 category, 1,000 patterns",
    "c1": "configs[1]: 128-tip pectinate rerooted vs original, GTR+G4, 10,000 patterns per GPU",
    "c2": "configs[2]: 1,024-tip Yule rerooted, GTR+G4, 100,000 patterns per GPU",
    "c2_paper": "1,024-tip paper-random (PAPER.md:148) rerooted, GTR+G4, 100,000 patterns per GPU",
    "c3": "configs[3]: 256-tip paper-random rerooted, GY94+G4 (61 states), 10,000 patterns per GPU",
    "c4": "configs[4]: 4,096-tip pectinate rerooted, GTR+G4, 4,194,304 patterns (strong scaling)",
}
METRIC = "updatePartials GFLOPS rerooted vs original root; %HBM roofline; 1/2/4/8 GPU"


def flops_per_pass(n, p, c, s):
    return (n - 1) * p * c * s * (4 * s - 1)


def bytes_per_pass(ops, n, p, c, s, elt, cumulative=True):
    """Algorithmic HBM bytes of all updatePartials launches of one pass
    (DESIGN.md §Roofline): per op and pattern, each internal child's c*s*elt
    partials (+4 B cumulative exponent), each tip child's 1 B state, the
    c*s*elt output and the 4 B exponent."""
    per = 0
    for o in ops:
        for ch in (int(o["child1"]), int(o["child2"])):
            per += 1 if ch < n else c * s * elt + (4 if cumulative else 0)
        per += c * s * elt + 4
    return per * p


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


# ----------------------------------------------------------------------------- helpers
def rank_workload(cfg: str, rank: int, world: int, seed: int = 1):
    """Weak scaling (c0-c2): each rank owns patterns [r p, (r+1) p) of a global
    alignment of world*p patterns.  Strong scaling (c4): the global p is split."""
    base = dict(CONFIGS[cfg])
    p = base["p"]
    if cfg == "c4":
        chunk = math.ceil(p / world)
        lo, hi = rank * chunk, min(p, (rank + 1) * chunk)
        w = config_workload(cfg, seed=seed, p=1)           # tree + model only
        rng = np.random.default_rng(np.random.SeedSequence([seed, 7919, rank]))
        w.tips = rng.integers(0, w.s, size=(w.n, hi - lo), dtype=np.uint8)
        w.pattern_weights = np.ones(hi - lo)
        return w, "strong"
    w = config_workload(cfg, seed=seed, p=p * world)
    w.tips = np.ascontiguousarray(w.tips[:, rank * p:(rank + 1) * p])
    w.pattern_weights = np.ones(p)
    return w, "weak"


def ncu_traffic(cfg: str, precision: int):
    """DRAM bytes per updatePartials launch from the committed ncu capture
    (profiles/ncu_traffic.json); null when there is none for this config."""
    path = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    try:
        d = json.load(open(path))
        return d.get(f"{cfg}_fp{precision}")
    except Exception:
        return None


def measured_peaks():
    try:
        return json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json"))), "measured"
    except Exception:
        return {"hbm_gbs": 6650.0}, "fallback"


# ----------------------------------------------------------------------------- reference arm
def run_reference(args, rank, world):
    """--impl reference: the fp64 oracle (test infrastructure) timed as it
    stands on the host cores, on a bounded pattern sample of the workload."""
    if rank != 0:
        return
    from threadpoolctl import threadpool_limits

    from oracle import model as om, pruning
    w, _ = rank_workload(args.config, 0, 1)
    sample = min(w.p, args.ref_patterns)
    tips = np.ascontiguousarray(w.tips[:, :sample])
    pw = np.ones(sample)
    Q = om.rate_matrix(w.model)
    fl = flops_per_pass(w.n, sample, w.c, w.s)
    with threadpool_limits(limits=1):
        t0 = time.perf_counter()
        pruning.prune(w.tree, Q, w.model.pi, w.rates, w.cat_weights, tips, pw)
        est = (time.perf_counter() - t0) * (args.steps + args.warmup)
        if est > 150.0:  # keep the whole reference run within a few minutes
            sample = max(256, int(sample * 150.0 / est))
            tips = np.ascontiguousarray(w.tips[:, :sample])
            pw = np.ones(sample)
            fl = flops_per_pass(w.n, sample, w.c, w.s)
        for _ in range(args.warmup):
            pruning.prune(w.tree, Q, w.model.pi, w.rates, w.cat_weights, tips, pw)
        t0 = time.perf_counter()
        for _ in range(args.steps):
            pruning.prune(w.tree, Q, w.model.pi, w.rates, w.cat_weights, tips, pw)
        dt = time.perf_counter() - t0
    val = fl * args.steps / dt / 1e9
    line = {
        "impl": "reference", "metric": METRIC, "value": val, "unit": "GFLOPS",
        "n_gpus": world, "steps": args.steps, "warmup": args.warmup,
        "ms_per_step": dt / args.steps * 1e3, "higher_is_better": True, "scaling": "weak",
        "vs_baseline": None, "dtype": "f64", "data": "synthetic (seeded, workloads/)",
        "config": {"workload": CONFIG_DESC.get(args.config, args.config),
                   "sample_patterns": sample, "schedule": "post-order (oracle)"},
        "cpu_baseline": {"value": val, "unit": "GFLOPS", "cores": 1, "kind": "oracle",
                         "sample": f"{sample} of {w.p} patterns, full {w.n}-tip tree, per step"},
        "e2e": {"value": val, "unit": "GFLOPS", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)


def cpu_baseline(w, budget_s=15.0):
    """The oracle as it stands on one host core, on a bounded pattern sample."""
    from threadpoolctl import threadpool_limits

    from oracle import model as om, pruning
    Q = om.rate_matrix(w.model)
    sample = min(w.p, 2000)
    tips = np.ascontiguousarray(w.tips[:, :sample])
    pw = np.ones(sample)
    reps, t_total = 0, 0.0
    with threadpool_limits(limits=1):
        while t_total < budget_s and reps < 50:
            t0 = time.perf_counter()
            pruning.prune(w.tree, Q, w.model.pi, w.rates, w.cat_weights, tips, pw)
            t_total += time.perf_counter() - t0
            reps += 1
    val = flops_per_pass(w.n, sample, w.c, w.s) * reps / t_total / 1e9
    return {"value": val, "unit": "GFLOPS", "cores": 1, "kind": "oracle",
            "sample": f"{reps} passes x {sample} of {w.p} patterns, full {w.n}-tip tree "
                      f"({t_total:.1f} s, numpy/scipy fp64, 1 thread)"}


# ----------------------------------------------------------------------------- our arm
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
                    help="skip the configs[2] HBM-regime measurement that rides along with c1")
    ap.add_argument("--no-fused", action="store_true",
                    help="skip the one-launch-per-pass (RRL_FLAG_FUSED_PASS) measurement")
    ap.add_argument("--ref-patterns", type=int, default=10_000)
    args = ap.parse_args()
    args.warmup = max(args.warmup, 3)

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
    # a dedicated (capturable, non-legacy) stream for everything timed below
    torch.cuda.set_stream(torch.cuda.Stream())
    dist = None
    backend = os.environ.get("RRL_DIST_BACKEND", "nccl")  # gloo: CPU-side test of the wiring
    if world > 1:
        import torch.distributed as dist
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
        else:
            dist.init_process_group(backend)

    def allreduce_(t, op=None):
        """In-place all-reduce of a device tensor (NCCL on the device; gloo via host)."""
        op = dist.ReduceOp.SUM if op is None else op
        if backend == "nccl":
            dist.all_reduce(t, op=op)
        else:
            h = t.cpu()
            dist.all_reduce(h, op=op)
            t.copy_(h)

    from paper_conf_ipps_ayresc18_b200 import build as _b
    _b.build()
    from paper_conf_ipps_ayresc18_b200 import TreeLikelihood, rrl as R

    stream = torch.cuda.current_stream()
    flush = torch.empty(512 * 1024 * 1024 // 4, dtype=torch.float32, device="cuda")
    d_out = torch.zeros(1, dtype=torch.float64, device="cuda")
    peaks, peak_src = measured_peaks()
    hbm = float(peaks.get("hbm_gbs", 6650.0))

    def maxall(x):
        if dist is None:
            return x
        t = torch.tensor([x], dtype=torch.float64, device="cuda")
        allreduce_(t, dist.ReduceOp.MAX)
        return float(t.item())

    def make(w, mode, precision, reuse, fused=False):
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
            allreduce_(d_out)

    def timed(tl, steps, warmup, clocks=None):
        """Per-step CUDA events on the launching stream; L2 flushed before
        every step outside the events; barrier + synchronize on both sides."""
        for _ in range(warmup):
            flush.zero_()
            step(tl)
        torch.cuda.synchronize()
        if dist is not None:
            dist.barrier()
        torch.cuda.synchronize()
        evs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True))
               for _ in range(steps)]
        # library profiling: CUDA events on this stream around every graph
        # replay of the updatePartials region (the roofline's launch durations)
        R.rrl_set_profiling(tl.inst, True)
        R.rrl_reset_profile(tl.inst)
        for i, (a, b) in enumerate(evs):
            flush.zero_()
            a.record(stream)
            step(tl)
            b.record(stream)
            if clocks is not None and i % 16 == 15:
                clocks.sample()  # the GPU is still running enqueued steps
        if clocks is not None:
            clocks.sample()
        torch.cuda.synchronize()
        if dist is not None:
            dist.barrier()
        torch.cuda.synchronize()
        ms = sum(a.elapsed_time(b) for a, b in evs)
        prof = R.rrl_get_profile(tl.inst)
        R.rrl_set_profiling(tl.inst, False)
        return maxall(ms), prof

    def measure(cfg, precision, steps, warmup, with_original=True, keep=False):
        w, scaling = rank_workload(cfg, rank, world)
        n, p, c, s = w.n, w.p, w.c, w.s
        elt = 4 if precision == 32 else 8
        reuse = cfg == "c4"
        tl = make(w, "reroot", precision, reuse)
        sched = tl.sched
        clocks = ClockSampler(local)
        ms, prof = timed(tl, steps, warmup, clocks)
        launches = prof["kernel_launches"]
        clk = clocks.stop()
        fl = flops_per_pass(n, p, c, s)
        nsi = steps
        part_ms = maxall(prof["partials_ms"]) / nsi
        bpp = bytes_per_pass(sched["ops"], n, p, c, s, elt)
        achieved = bpp / (part_ms * 1e-3) / 1e9
        res = {
            "cfg": cfg, "w": w, "scaling": scaling, "n": n, "p": p, "c": c, "s": s,
            "value": fl * world * steps / (ms * 1e-3) / 1e9, "ms_per_step": ms / steps,
            "launches": launches, "clocks": clk, "sets": sched["set_count"], "fl": fl,
            "updatePartials": {"ms_per_pass": part_ms,
                               "launches_per_pass": prof["partials_launches"] / nsi,
                               "gflops": fl / (part_ms * 1e-3) / 1e9,
                               "pattern_node_updates_per_s": (n - 1) * p / (part_ms * 1e-3),
                               "share_of_step": part_ms / (ms / steps)},
            "roofline": {"bound": "hbm", "achieved": achieved, "peak": hbm, "unit": "GB/s",
                         "frac": achieved / hbm, "traffic": ncu_traffic(cfg, precision),
                         "kernel": "k_partials_nuc / k_partials_nuc_bulk (updatePartials, one "
                                   "launch per level set)",
                         "algorithmic_bytes_per_pass": bpp,
                         "algorithmic_bytes_per_launch": bpp / max(1.0, prof["partials_launches"] / nsi),
                         "launches_per_pass": prof["partials_launches"] / nsi,
                         "peak_source": f"{peak_src} hbm_gbs (MEASURED_PEAKS.json)",
                         "timing": "CUDA events on the launching stream around every CUDA-graph "
                                   "replay of the updatePartials region inside the timed steps; "
                                   "per-launch duration = region time / level-set launches"},
            "lnL": float(d_out.item()),
        }
        if s == 61 and precision == 32:
            # tcgen05 codon kernel: HBM-bound once the tensor cores carry the
            # contraction; algorithmic bytes count 61 states (the 64-wide
            # padding is overhead).  Tensor work for context.
            res["roofline"]["tensor_tflops"] = fl / (part_ms * 1e-3) / 1e12
            res["roofline"]["kernel"] = ("k_partials_codon_tc5 (TMA-fed tcgen05 kind::tf32, 3xTF32)"
                                         if os.environ.get("RRL_CODON_TC5", "1") != "0" else
                                         "k_partials_codon_tc (tcgen05 kind::tf32, 3xTF32)")
        if s == 61 and precision == 64:
            # SIMT fp64 codon kernel: bound by FP64 FMA issue, not HBM
            peak_tf = 148 * 64 * 2 * 1.965e9 / 1e12
            ach = fl / (part_ms * 1e-3) / 1e12
            res["roofline"].update({
                "bound": "alu", "achieved": ach, "peak": peak_tf, "unit": "TFLOP/s",
                "frac": ach / peak_tf, "hbm_achieved_gbs": achieved,
                "peak_source": "derived: 148 SMs x 64 FP64 lanes x 2 flop x 1.965 GHz "
                               "(B200_PROFILING.md clocks; DESIGN.md §6)",
                "flops": "effective Eq.(1) flops (n-1) c s (4s-1) per pattern (reading A16)"})
        if with_original and cfg != "c4":
            to = make(w, "level", precision, False)
            ms_o, prof_o = timed(to, steps, warmup)
            po = maxall(prof_o["partials_ms"]) / nsi
            res["reroot"] = {
                "sets": sched["set_count"], "sets_original": to.sched["set_count"],
                "theoretical_speedup": to.sched["set_count"] / sched["set_count"],
                "step_speedup": ms_o / ms, "updatePartials_speedup": po / part_ms,
                "original_gflops": fl * world * steps / (ms_o * 1e-3) / 1e9,
                "paper_context": "BEAGLE CUDA on Quadro GP100: up to 1.93x (pectinate, 406 OTUs, "
                                 "512 patterns, PAPER.md:258); mean 1.26x (random 256 OTUs, "
                                 "PAPER.md:230)"}
            to.close()
        if s == 4 and cfg != "c4" and not args.no_fused:
            # RRL_FLAG_FUSED_PASS (beyond the paper): the whole
            # pass as ONE launch; level sets still bound its dependent chain.
            fused = {}
            for mode in ("reroot", "level"):
                tf = make(w, mode, precision, False, fused=True)
                ms_f, prof_f = timed(tf, steps, warmup)
                pf = maxall(prof_f["partials_ms"]) / nsi
                fused[mode] = {"value": fl * world * steps / (ms_f * 1e-3) / 1e9,
                               "ms_per_step": ms_f / steps, "updatePartials_ms_per_pass": pf,
                               "launches_per_pass": prof_f["partials_launches"] / nsi,
                               "hbm_gbs": bpp / (pf * 1e-3) / 1e9,
                               "lnL": float(d_out.item())}
                tf.close()
            res["fused_pass"] = {
                "kernel": "k_partials_nuc_fused (RRL_FLAG_FUSED_PASS: one launch per pass)",
                "value": fused["reroot"]["value"], "unit": "GFLOPS",
                "ms_per_step": fused["reroot"]["ms_per_step"],
                "updatePartials_ms_per_pass": fused["reroot"]["updatePartials_ms_per_pass"],
                "roofline_frac": fused["reroot"]["hbm_gbs"] / hbm,
                "reroot_vs_original_updatePartials": fused["level"]["updatePartials_ms_per_pass"]
                / fused["reroot"]["updatePartials_ms_per_pass"],
                "original": fused["level"], "lnL": fused["reroot"]["lnL"]}
        if keep:
            res["tl"] = tl
        else:
            tl.close()
        return res

    prim = measure(args.config, args.precision, args.steps, args.warmup, keep=True)
    w, tl = prim["w"], prim["tl"]
    n, p = prim["n"], prim["p"]

    # ---- e2e through the public API with host buffers (pinned), every step:
    # reroot + schedule, H2D tips + branch lengths, pass, D2H of the lnL.
    reuse = args.config == "c4"
    pinned = torch.empty(w.tips.shape, dtype=torch.uint8, pin_memory=True).numpy()
    pinned[:] = w.tips
    e2e_steps = max(3, min(args.steps, 50))
    for _ in range(2):
        tl.set_tips(pinned)
        tl.set_tree(w.tree.parent, w.tree.blen, "reroot", reuse_buffers=reuse)
        tl.loglik()
    torch.cuda.synchronize()
    if dist is not None:
        dist.barrier()
    t0 = time.perf_counter()
    for _ in range(e2e_steps):
        tl.set_tips(pinned)
        tl.set_tree(w.tree.parent, w.tree.blen, "reroot", reuse_buffers=reuse)
        tl.update()
        tl.root_loglik_device(d_out.data_ptr())
        if dist is not None:
            allreduce_(d_out)
        float(d_out.item())
    e2e_s = maxall(time.perf_counter() - t0)
    e2e_val = prim["fl"] * world * e2e_steps / e2e_s / 1e9
    h2d = int(w.tips.nbytes + tl.t.nbytes + tl.matrix_idx.nbytes)
    tl.close()

    # ---- the HBM-bound regime (configs[2]) beside the launch-bound headline
    sec = None
    if args.config == "c1" and not args.no_secondary:
        sec = measure("c2", args.precision, min(args.steps, 30), args.warmup)

    if rank != 0:
        if dist is not None:
            dist.destroy_process_group()
        return
    cpu = None if args.no_cpu_baseline else cpu_baseline(w)
    out = {
        "metric": METRIC,
        "value": prim["value"],
        "unit": "GFLOPS",
        "n_gpus": world,
        "steps": args.steps,
        "warmup": args.warmup,
        "ms_per_step": prim["ms_per_step"],
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
                "path": "TreeLikelihood: set_tips (pinned H2D) + rrl_reroot_and_schedule + K1 + "
                        "level-set K2 + K4 + D2H lnL"},
        "gpu_launches": int(prim["launches"]),
        "clocks": prim["clocks"],
        "lnL": prim["lnL"],
    }
    if "fused_pass" in prim:
        out["fused_pass"] = prim["fused_pass"]
    if sec is not None:
        out["hbm_regime"] = {
            "workload": CONFIG_DESC["c2"], "value": sec["value"], "unit": "GFLOPS",
            "ms_per_step": sec["ms_per_step"], "reroot": sec.get("reroot"),
            "updatePartials": sec["updatePartials"], "roofline": sec["roofline"],
            "gpu_launches": int(sec["launches"]), "clocks": sec["clocks"]}
        if "fused_pass" in sec:
            out["hbm_regime"]["fused_pass"] = sec["fused_pass"]
    print(json.dumps(out), flush=True)
    if dist is not None:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
