#!/usr/bin/env python3
"""Reroot-speedup and HBM-fraction sweeps on one B200.

    python tools/reroot_sweep.py [--out gpurun_out/sweep.json] [--quick]

Part A (§8(d)-5): 1,024-tip pectinate, GTR+G4, fp32 and fp64, patterns in
{512, 1K, 2K, 4K, 10K, 100K, 1M}: original-root (1,023 sets) vs rerooted (512
sets) level-set schedules, timed interleaved with an identical-schedule
control arm.  Reports, per point, the updatePartials time (CUDA events on the
launching stream around each CUDA-graph replay of all level-set launches; L2
flushed before every rep; median and best), the reroot speedup S = T_orig /
T_reroot against the bound 1,023/512 and against the NEXT-4 cost model's
prediction, and the algorithmic-HBM fractions.

Part B (the paper's own experiments) now lives in tools/paper_experiments.py.

Part C (NEXT-4): host cost of the O(n) rerooting DP and of the paper's
exhaustive O(n^2) search (C++) against the per-pass time rerooting saves
(PAPER.md:270, 288).
"""
from __future__ import annotations

import argparse
import json
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--out", default=os.path.join(ROOT, "gpurun_out", "sweep.json"))
    ap.add_argument("--quick", action="store_true")
    ap.add_argument("--reps", type=int, default=20)
    args = ap.parse_args()

    import torch
    torch.cuda.set_device(0)
    torch.cuda.set_stream(torch.cuda.Stream())
    stream = torch.cuda.current_stream()
    from paper_conf_ipps_ayresc18_b200 import build
    build.build()
    from paper_conf_ipps_ayresc18_b200 import TreeLikelihood, rrl as R
    from workloads import make_workload
    hbm = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))["hbm_gbs"]
    flush = torch.empty(512 * 1024 * 1024 // 4, dtype=torch.float32, device="cuda")

    def make(w, mode, precision, reuse=True):
        nbuf = R.rrl_reroot_and_schedule(w.n, w.tree.parent, w.tree.blen, mode, reuse)["buffer_count"]
        tl = TreeLikelihood(w.n, w.p, w.s, w.c, precision=precision, cuda_graph=True,
                            buffer_count=nbuf, stream_ptr=stream.cuda_stream)
        tl.set_model_params(w.model, w.rates, w.cat_weights)
        tl.set_tips(w.tips)
        tl.set_tree(w.tree.parent, w.tree.blen, mode, reuse_buffers=reuse)
        for _ in range(3):
            tl.update()
        R.rrl_set_profiling(tl.inst, True)
        return tl

    def interleaved(arms, reps):
        """Arms timed rep by rep (drifts hit every arm alike); updatePartials
        region per rep, L2 flushed before every rep."""
        t = [[] for _ in arms]
        for _ in range(reps):
            for i, a in enumerate(arms):
                flush.zero_()
                R.rrl_reset_profile(a.inst)
                a.update()
                t[i].append(R.rrl_get_profile(a.inst)["partials_ms"])
        return [(float(np.median(x)), float(min(x))) for x in t]

    def alg_bytes(tl, w, elt):
        per = 0
        for o in tl.sched["ops"]:
            for ch in (int(o["child1"]), int(o["child2"])):
                per += 1 if ch < w.n else w.c * 4 * elt + 4
            per += w.c * 4 * elt + 4
        return per * w.p

    out = {"hbm_gbs_measured": hbm, "time": time.time(), "partA": [],
           "method": "interleaved arms (original, rerooted, identical-schedule control), median and best of "
                     "the reps, updatePartials region only, L2 flushed before every rep; predicted = "
                     "rrl_schedule_cost (t0 2 us, 0.95 x measured HBM, 126 MB L2)"}
    # ---------------- Part A
    pats = [512, 1024, 2048, 4096, 10_000, 100_000, 1_000_000]
    if args.quick:
        pats = [512, 10_000, 100_000]
    for precision in (32, 64):
        elt = 4 if precision == 32 else 8
        for p in pats:
            w = make_workload(tree_kind="pectinate", n=1024, p=p, model="gtr", c=4, seed=1)
            reps = args.reps if p < 1_000_000 else 5
            arms = [make(w, "level", precision), make(w, "reroot", precision), make(w, "level", precision)]
            (mo, bo), (mr, br), (mc, _) = interleaved(arms, reps)
            pred = [R.rrl_schedule_cost(1024, a.sched["ops"], a.sched["set_offsets"], p, 4, 4, precision,
                                        2.0, 0.95 * hbm, 126e6) for a in arms[:2]]
            row = {"precision": precision, "patterns": p, "reps": reps,
                   "sets_original": arms[0].sched["set_count"], "sets_reroot": arms[1].sched["set_count"],
                   "bound": arms[0].sched["set_count"] / arms[1].sched["set_count"],
                   "orig_ms_median": mo, "reroot_ms_median": mr, "orig_ms_best": bo, "reroot_ms_best": br,
                   "speedup_median": mo / mr, "speedup_best": bo / br, "control_ratio": mo / mc,
                   "predicted_speedup": pred[0] / pred[1],
                   "reroot_hbm_frac": alg_bytes(arms[1], w, elt) / (mr * 1e-3) / 1e9 / hbm,
                   "orig_hbm_frac": alg_bytes(arms[0], w, elt) / (mo * 1e-3) / 1e9 / hbm}
            for a in arms:
                a.close()
            out["partA"].append(row)
            print(json.dumps(row), flush=True)

    # Part B (the paper's experiments at 512 patterns) moved to tools/paper_experiments.py.
    def run(w, mode, precision, reps):
        tl = make(w, mode, precision, reuse=False)
        (m, b), = interleaved([tl], reps)
        tl.close()
        return {"mean_ms": m, "best_ms": b}

    # ---------------- Part C (NEXT-4): cost of rerooting vs its benefit
    C = []
    for kind in ("random", "pectinate"):
        for n in (64, 256, 1024, 4096):
            w = make_workload(tree_kind=kind, n=n, p=512, model="gtr", c=4, seed=1)
            reps = 20
            t0 = time.perf_counter()
            for _ in range(reps):
                R.rrl_reroot_and_schedule(n, w.tree.parent, w.tree.blen, "reroot")
            dp_ms = (time.perf_counter() - t0) / reps * 1e3
            t0 = time.perf_counter()
            R.rrl_reroot_exhaustive(n, w.tree.parent, w.tree.blen)
            ex_ms = (time.perf_counter() - t0) * 1e3
            o = run(w, "level", 32, 10)
            r = run(w, "reroot", 32, 10)
            saved = o["mean_ms"] - r["mean_ms"]
            row = {"kind": kind, "n": n, "patterns": 512, "dp_reroot_schedule_ms": dp_ms,
                   "exhaustive_cpp_ms": ex_ms, "pass_orig_ms": o["mean_ms"], "pass_reroot_ms": r["mean_ms"],
                   "saved_per_pass_ms": saved,
                   "breakeven_passes_dp": (dp_ms / saved) if saved > 0 else None,
                   "breakeven_passes_exhaustive": (ex_ms / saved) if saved > 0 else None}
            C.append(row)
            print(json.dumps(row), flush=True)
    out["partC_reroot_cost"] = C
    os.makedirs(os.path.dirname(args.out), exist_ok=True)
    json.dump(out, open(args.out, "w"), indent=1)


if __name__ == "__main__":
    main()
