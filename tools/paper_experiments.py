#!/usr/bin/env python3
"""The paper's experiments re-run on one B200 (run under gpurun).

    python tools/paper_experiments.py [--out gpurun_out/paper_experiments.json] [--trees 1000]

All at 512 site patterns, GTR+G4, fp32, rescaling every pass,
updatePartials time only (CUDA events around each CUDA-graph replay of the
level-set launches, reading A17), L2 flushed before every rep.  Arms of one
comparison are timed interleaved (rep by rep) and reported as the median over
the reps (and best), so clock drift hits every arm alike.

* Table III: 64 OTUs -- balanced, pectinate, pectinate
  rerooted, 100 paper-random trees +- reroot: concurrency speedup over the
  sequential one-operation-per-launch schedule, against the theoretical
  63 / sets; plus an identical-schedule control (pectinate LEVEL vs
  SEQUENTIAL, which are the same 63 launches).
* the 406-OTU pectinate tree (1.93x on GP100).
* Fig. 4 / Fig. 5: 100 paper-random 256-OTU trees, sets
  and throughput original vs rerooted (mean speedup 1.26x on GP100).
* Fig. 6: 16 ... 4,096 OTUs, balanced, pectinate and
  `--trees` paper-random trees per size, each original and rerooted:
  throughput distributions.
"""
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
    ap.add_argument("--out", default=os.path.join(ROOT, "gpurun_out", "paper_experiments.json"))
    ap.add_argument("--trees", type=int, default=1000, help="random trees per size in the Fig. 6 sweep")
    ap.add_argument("--reps", type=int, default=30)
    ap.add_argument("--budget-s", type=float, default=900.0, help="stop the Fig. 6 sweep's random trees early")
    args = ap.parse_args()

    import torch
    torch.cuda.set_device(0)
    torch.cuda.set_stream(torch.cuda.Stream())
    stream = torch.cuda.current_stream()
    from paper_conf_ipps_ayresc18_b200 import build
    build.build()
    from paper_conf_ipps_ayresc18_b200 import TreeLikelihood, rrl as R
    from workloads import make_workload
    flush = torch.empty(512 * 1024 * 1024 // 4, dtype=torch.float32, device="cuda")
    P = 512

    class Arm:
        """One instance per (tree, schedule); update() = K1 + the level-set launches."""

        def __init__(self, w, mode, tl=None):
            self.tl = tl or TreeLikelihood(w.n, w.p, w.s, w.c, precision=32, cuda_graph=True,
                                           stream_ptr=stream.cuda_stream)
            if tl is None:
                self.tl.set_model_params(w.model, w.rates, w.cat_weights)
                self.tl.set_tips(w.tips)
            self.tl.set_tree(w.tree.parent, w.tree.blen, mode)
            self.sets = self.tl.sched["set_count"]
            for _ in range(2):
                self.tl.update()
            R.rrl_set_profiling(self.tl.inst, True)

        def time(self):
            flush.zero_()
            R.rrl_reset_profile(self.tl.inst)
            self.tl.update()
            return R.rrl_get_profile(self.tl.inst)["partials_ms"]

    def interleaved(arms, reps):
        t = [[] for _ in arms]
        for _ in range(reps):
            for i, a in enumerate(arms):
                t[i].append(a.time())
        return [{"median_ms": float(np.median(x)), "best_ms": float(min(x))} for x in t]

    def gflops(n, ms):
        return (n - 1) * P * 4 * 4 * 15 / (ms * 1e-3) / 1e9

    out = {"patterns": P, "reps": args.reps, "method": "interleaved arms, median (and best) over reps, "
           "updatePartials region only, L2 flushed before every rep"}
    t_start = time.time()

    # ------------------------------------------------ Table III (64 OTUs)
    t3 = {}
    for kind in ("balanced", "pectinate"):
        w = make_workload(tree_kind=kind, n=64, p=P, model="gtr", c=4, seed=1)
        arms = [Arm(w, "sequential"), Arm(w, "level"), Arm(w, "reroot"), Arm(w, "sequential")]
        st = interleaved(arms, args.reps * 3)
        seq = st[0]["median_ms"]
        t3[kind] = {"sets": arms[1].sets, "theory": 63 / arms[1].sets,
                    "speedup_vs_sequential": seq / st[1]["median_ms"],
                    "control_identical_sequential_ratio": seq / st[3]["median_ms"]}
        t3[kind + "_rerooted"] = {"sets": arms[2].sets, "theory": 63 / arms[2].sets,
                                  "speedup_vs_sequential": seq / st[2]["median_ms"]}
        for a in arms:
            a.tl.close()
    for name, mode in (("random", "level"), ("random_rerooted", "reroot")):
        rows = []
        for seed in range(1, 101):
            w = make_workload(tree_kind="random", n=64, p=P, model="gtr", c=4, seed=seed)
            arms = [Arm(w, "sequential"), Arm(w, mode)]
            st = interleaved(arms, args.reps)
            rows.append((63 / arms[1].sets, st[0]["median_ms"] / st[1]["median_ms"]))
            for a in arms:
                a.tl.close()
        a = np.array(rows)
        t3[name] = {"theory_range": [float(a[:, 0].min()), float(a[:, 0].max())],
                    "speedup_range": [float(a[:, 1].min()), float(a[:, 1].max())],
                    "realized_mean": float((a[:, 1] / a[:, 0]).mean()),
                    "within_theory": int((a[:, 1] <= a[:, 0] * 1.02).sum()), "trees": len(rows)}
    out["table3_64otu"] = t3
    print(json.dumps(t3), flush=True)

    # ------------------------------------------------ PAPER.md:258, 406-OTU pectinate
    w = make_workload(tree_kind="pectinate", n=406, p=P, model="gtr", c=4, seed=1)
    arms = [Arm(w, "level"), Arm(w, "reroot")]
    st = interleaved(arms, args.reps * 3)
    out["pectinate_406"] = {"sets": [a.sets for a in arms], "gflops": [gflops(406, s["median_ms"]) for s in st],
                            "speedup": st[0]["median_ms"] / st[1]["median_ms"], "bound": arms[0].sets / arms[1].sets,
                            "paper": "1.93x on Quadro GP100 (PAPER.md:258)"}
    for a in arms:
        a.tl.close()
    print(json.dumps(out["pectinate_406"]), flush=True)

    # ------------------------------------------------ Fig. 4 / 5: 100 random 256-OTU trees
    f45 = []
    for seed in range(1, 101):
        w = make_workload(tree_kind="random", n=256, p=P, model="gtr", c=4, seed=seed)
        arms = [Arm(w, "level"), Arm(w, "reroot")]
        st = interleaved(arms, args.reps)
        f45.append({"seed": seed, "sets": [a.sets for a in arms], "gflops": [gflops(256, s["median_ms"]) for s in st],
                    "speedup": st[0]["median_ms"] / st[1]["median_ms"]})
        for a in arms:
            a.tl.close()
    sp = np.array([x["speedup"] for x in f45])
    out["fig4_fig5_256otu"] = {"trees": f45, "mean_speedup": float(sp.mean()),
                               "max_set_reduction": float(max(x["sets"][0] / x["sets"][1] for x in f45)),
                               "unchanged_trees": int(sum(x["sets"][0] == x["sets"][1] for x in f45)),
                               "paper": "mean 1.26x on Quadro GP100 (PAPER.md:230); sets reduced by up to half, "
                                        "one of 100 trees unchanged (PAPER.md:205)"}
    print(json.dumps({k: v for k, v in out["fig4_fig5_256otu"].items() if k != "trees"}), flush=True)

    # ------------------------------------------------ Fig. 6: 16 ... 4,096 OTUs
    fig6 = []
    sizes = [16, 32, 64, 128, 256, 512, 1024, 2048, 4096]
    per_size_budget = args.budget_s / len(sizes)
    for n in sizes:
        row = {"otus": n}
        for kind in ("balanced", "pectinate"):
            w = make_workload(tree_kind=kind, n=n, p=P, model="gtr", c=4, seed=1)
            arms = [Arm(w, "level"), Arm(w, "reroot")]
            st = interleaved(arms, args.reps)
            row[kind] = {"sets": [a.sets for a in arms], "gflops": [gflops(n, s["median_ms"]) for s in st],
                         "speedup": st[0]["median_ms"] / st[1]["median_ms"]}
            for a in arms:
                a.tl.close()
        # random trees: one instance per arm, re-used across trees (set_tree per tree)
        w0 = make_workload(tree_kind="random", n=n, p=P, model="gtr", c=4, seed=1)
        base = [None, None]
        g_o, g_r, s_o, s_r = [], [], [], []
        t0 = time.time()
        for seed in range(1, args.trees + 1):
            w = make_workload(tree_kind="random", n=n, p=P, model="gtr", c=4, seed=seed)
            w.tips, w.model, w.rates = w0.tips, w0.model, w0.rates
            arms = [Arm(w, "level", base[0]), Arm(w, "reroot", base[1])]
            base = [arms[0].tl, arms[1].tl]
            st = interleaved(arms, max(5, args.reps // 3))
            g_o.append(gflops(n, st[0]["median_ms"]))
            g_r.append(gflops(n, st[1]["median_ms"]))
            s_o.append(arms[0].sets)
            s_r.append(arms[1].sets)
            if time.time() - t0 > per_size_budget:
                break
        for b in base:
            b.close()

        def q(x):
            return [float(v) for v in np.percentile(np.array(x), [0, 25, 50, 75, 100])]
        row["random"] = {"trees": len(g_o), "gflops_original_q": q(g_o), "gflops_rerooted_q": q(g_r),
                         "sets_original_q": q(s_o), "sets_rerooted_q": q(s_r),
                         "speedup_mean": float(np.mean(np.array(g_r) / np.array(g_o)))}
        fig6.append(row)
        print(json.dumps(row), flush=True)
    out["fig6_sizes"] = fig6
    out["elapsed_s"] = time.time() - t_start
    os.makedirs(os.path.dirname(args.out), exist_ok=True)
    json.dump(out, open(args.out, "w"), indent=1)


if __name__ == "__main__":
    main()
