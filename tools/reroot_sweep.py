#!/usr/bin/env python3
"""Reroot-speedup and HBM-fraction sweeps on one B200.

    python tools/reroot_sweep.py [--out gpurun_out/sweep.json] [--quick]

Part A (§8(d)-5): 1,024-tip pectinate, GTR+G4, fp32 and fp64, patterns in
{512, 1K, 2K, 4K, 10K, 100K, 1M}: original-root (1,023 sets) vs rerooted (512
sets) level-set schedules.  Reports, per point, the updatePartials time (CUDA
events on the launching stream around each CUDA-graph replay of all level-set
launches; L2 flushed before every replay), the
reroot speedup S = T_orig / T_reroot against the bound 1,023/512, and the
rerooted algorithmic-HBM fraction.

Part B (NEXT-1, the paper's own experiments re-run on B200): 512 patterns
(PAPER.md:180), fp32 with rescaling: Table III (64 OTUs: balanced, pectinate,
pectinate rerooted, 100 paper-random trees +- reroot; concurrency speedup over
the sequential one-op-per-launch schedule), the 406-OTU pectinate point of
PAPER.md:258 (best 1.93x on GP100), and Fig. 4/5 (100 paper-random 256-OTU
trees: sets and throughput original vs rerooted; mean speedup 1.26x on GP100,
PAPER.md:230).

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

    def run(w, mode, precision, reps, reuse=True):
        nbuf = R.rrl_reroot_and_schedule(w.n, w.tree.parent, w.tree.blen, mode, reuse)["buffer_count"]
        tl = TreeLikelihood(w.n, w.p, w.s, w.c, precision=precision, cuda_graph=True,
                            buffer_count=nbuf, stream_ptr=stream.cuda_stream)
        tl.set_model_params(w.model, w.rates, w.cat_weights)
        tl.set_tips(w.tips)
        tl.set_tree(w.tree.parent, w.tree.blen, mode, reuse_buffers=reuse)
        for _ in range(3):
            tl.update()
        R.rrl_set_profiling(tl.inst, True)
        R.rrl_reset_profile(tl.inst)
        best = float("inf")
        tot = 0.0
        for _ in range(reps):
            flush.zero_()
            torch.cuda.synchronize()
            before = R.rrl_get_profile(tl.inst)["partials_ms"]
            tl.update()
            ms = R.rrl_get_profile(tl.inst)["partials_ms"] - before
            best = min(best, ms)
            tot += ms
        lnl = tl.root_loglik()
        elt = 4 if precision == 32 else 8
        ops = tl.sched["ops"]
        per = 0
        for o in ops:
            for ch in (int(o["child1"]), int(o["child2"])):
                per += 1 if ch < w.n else w.c * 4 * elt + 4
            per += w.c * 4 * elt + 4
        res = {"sets": tl.sched["set_count"], "best_ms": best, "mean_ms": tot / reps,
               "alg_bytes": per * w.p, "lnL": lnl}
        tl.close()
        return res

    out = {"hbm_gbs_measured": hbm, "time": time.time(), "partA": [], "partB": {}}
    # ---------------- Part A
    pats = [512, 1024, 2048, 4096, 10_000, 100_000, 1_000_000]
    if args.quick:
        pats = [512, 10_000, 100_000]
    for precision in (32, 64):
        for p in pats:
            w = make_workload(tree_kind="pectinate", n=1024, p=p, model="gtr", c=4, seed=1)
            reps = args.reps if p < 1_000_000 else 5
            o = run(w, "level", precision, reps)
            r = run(w, "reroot", precision, reps)
            row = {"precision": precision, "patterns": p, "sets_original": o["sets"],
                   "sets_reroot": r["sets"], "bound": o["sets"] / r["sets"],
                   "orig_ms": o["mean_ms"], "reroot_ms": r["mean_ms"],
                   "speedup_mean": o["mean_ms"] / r["mean_ms"],
                   "speedup_best": o["best_ms"] / r["best_ms"],
                   "reroot_hbm_frac": r["alg_bytes"] / (r["mean_ms"] * 1e-3) / 1e9 / hbm,
                   "orig_hbm_frac": o["alg_bytes"] / (o["mean_ms"] * 1e-3) / 1e9 / hbm,
                   "reroot_gflops": (1023 * p * 4 * 4 * 15) / (r["mean_ms"] * 1e-3) / 1e9,
                   "lnL_rel_diff": abs(o["lnL"] - r["lnL"]) / abs(o["lnL"])}
            out["partA"].append(row)
            print(json.dumps(row), flush=True)

    # ---------------- Part B (paper's experiments, 512 patterns, fp32)
    def tput(w, mode):
        r = run(w, mode, 32, args.reps)
        fl = (w.n - 1) * w.p * w.c * 4 * 15
        return r, fl / (r["mean_ms"] * 1e-3) / 1e9

    B = out["partB"]
    t3 = {}
    for kind in ("balanced", "pectinate"):
        w = make_workload(tree_kind=kind, n=64, p=512, model="gtr", c=4, seed=1)
        seq, _ = tput(w, "sequential")
        lev, _ = tput(w, "level")
        t3[kind] = {"sets": lev["sets"], "theory": 63 / lev["sets"],
                    "speedup_vs_sequential": seq["mean_ms"] / lev["mean_ms"]}
        if kind == "pectinate":
            rr, _ = tput(w, "reroot")
            t3["pectinate_rerooted"] = {"sets": rr["sets"], "theory": 63 / rr["sets"],
                                        "speedup_vs_sequential": seq["mean_ms"] / rr["mean_ms"]}
    rnd, rnd_rr = [], []
    ntrees = 20 if args.quick else 100
    for seed in range(1, ntrees + 1):
        w = make_workload(tree_kind="random", n=64, p=512, model="gtr", c=4, seed=seed)
        seq, _ = tput(w, "sequential")
        lev, _ = tput(w, "level")
        rr, _ = tput(w, "reroot")
        rnd.append((63 / lev["sets"], seq["mean_ms"] / lev["mean_ms"]))
        rnd_rr.append((63 / rr["sets"], seq["mean_ms"] / rr["mean_ms"]))
    for name, arr in (("random", rnd), ("random_rerooted", rnd_rr)):
        a = np.array(arr)
        t3[name] = {"theory_range": [float(a[:, 0].min()), float(a[:, 0].max())],
                    "speedup_range": [float(a[:, 1].min()), float(a[:, 1].max())],
                    "realized_mean": float((a[:, 1] / a[:, 0]).mean())}
    B["table3_64otu_512pat"] = t3
    print(json.dumps(t3), flush=True)

    w = make_workload(tree_kind="pectinate", n=406, p=512, model="gtr", c=4, seed=1)
    o, go = tput(w, "level")
    r, gr = tput(w, "reroot")
    B["pectinate_406_512pat"] = {"sets": [o["sets"], r["sets"]], "gflops": [go, gr],
                                 "speedup": o["mean_ms"] / r["mean_ms"],
                                 "paper": "1.93x on Quadro GP100 (PAPER.md:258)"}
    print(json.dumps(B["pectinate_406_512pat"]), flush=True)

    f45 = []
    for seed in range(1, ntrees + 1):
        w = make_workload(tree_kind="random", n=256, p=512, model="gtr", c=4, seed=seed)
        o, go = tput(w, "level")
        r, gr = tput(w, "reroot")
        f45.append({"seed": seed, "sets": [o["sets"], r["sets"]], "gflops": [go, gr],
                    "speedup": o["mean_ms"] / r["mean_ms"]})
    sp = np.array([x["speedup"] for x in f45])
    B["fig4_fig5_256otu_512pat"] = {"trees": f45, "mean_speedup": float(sp.mean()),
                                    "max_set_reduction": float(max(x["sets"][0] / x["sets"][1] for x in f45)),
                                    "paper": "mean 1.26x on Quadro GP100 (PAPER.md:230); sets reduced by "
                                             "up to half (PAPER.md:205)"}
    print(json.dumps({k: v for k, v in B["fig4_fig5_256otu_512pat"].items() if k != "trees"}), flush=True)
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
