#!/usr/bin/env python3
"""A search-like loop of topology moves with partial updates (SURVEY.md NEXT-2 /
NEXT-4; run under gpurun).

    python tools/search_loop.py [--out gpurun_out/search_loop.json] [--moves 400]

A random walk of SPR / NNI moves (readings A26, A27) on a tree; after every
move the likelihood is brought up to date by recomputing only the invalidated
nodes (rrl_schedule_update, reading A28) and the root lnL is evaluated.
Rerooting policies compared ("it is sufficient to reroot the
starting tree ... further balanced rerootings, later in the search process,
might result in further performance gains"):
  never      -- the original rooting throughout;
  start      -- the starting tree rerooted once (rrl_reroot_and_schedule);
  periodic   -- the current tree fully rerooted (and recomputed) every K moves;
  partial    -- every partial update rerooted on the edge that minimises its
                own level sets (rrl_schedule_update with RRL_SCHED_REROOT);
  auto       -- start + the cost model of rrl_schedule_cost decides, for every
                update, between the rerooted and the current-rooting schedule.
Reported per policy: updatePartials GPU time over the loop (CUDA events around
each level-set launch), the device span of each update (events before and
after the host scheduling + K1 + launches, i.e. what a search loop waits for),
level sets and operations launched, host scheduling time, and the final lnL
against a full pass on the final tree.
Each policy runs the same seeded sequence of random draws on its own current
rooting (statistically equivalent walks).
"""
import argparse
import json
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def children(parent):
    ch = [[] for _ in range(len(parent))]
    for v, u in enumerate(parent):
        if u >= 0:
            ch[u].append(v)
    return ch


def random_move(R, n, parent, blen, rng):
    """One legal SPR or NNI on the current rooted tree (C++ moves)."""
    N = 2 * n - 1
    root = int(np.flatnonzero(parent < 0)[0])
    ch = children(parent)
    while True:
        if rng.random() < 0.5:
            x = int(rng.integers(0, N))
            if x == root or parent[x] == root:
                continue
            sub, st = set(), [x]
            while st:
                v = st.pop()
                sub.add(v)
                st.extend(ch[v])
            r = int(rng.integers(0, N))
            if r in sub or r == parent[x] or r == root:
                continue
            return R.rrl_tree_spr(n, parent, blen, x, r)
        v = int(rng.integers(n, N))
        if v == root:
            continue
        u = int(parent[v])
        if u == root:
            a, b = sorted(ch[root])
            if v != a or b < n:
                continue
        return R.rrl_tree_nni(n, parent, blen, v, int(rng.integers(0, 2)))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--out", default=os.path.join(ROOT, "gpurun_out", "search_loop.json"))
    ap.add_argument("--moves", type=int, default=400)
    ap.add_argument("--period", type=int, default=50)
    args = ap.parse_args()

    import torch
    torch.cuda.set_device(0)
    torch.cuda.set_stream(torch.cuda.Stream())
    stream = torch.cuda.current_stream()
    from paper_conf_ipps_ayresc18_b200 import build
    build.build()
    from paper_conf_ipps_ayresc18_b200 import TreeLikelihood, rrl as R
    from workloads import make_workload

    results = []
    for kind, n, p in (("pectinate", 1024, 512), ("random", 1024, 512), ("random", 1024, 10_000),
                       ("pectinate", 256, 100_000)):
        w = make_workload(tree_kind=kind, n=n, p=p, model="gtr", c=4, seed=1)
        row = {"tree": kind, "otus": n, "patterns": p, "moves": args.moves, "policies": {}}
        for policy in ("never", "start", "periodic", "partial", "auto"):
            tl = TreeLikelihood(n, p, 4, 4, precision=32, stream_ptr=stream.cuda_stream)
            tl.set_model_params(w.model, w.rates, w.cat_weights)
            tl.set_tips(w.tips)
            tl.set_tree(w.tree.parent, w.tree.blen, "level" if policy == "never" else "reroot")
            tl.loglik()
            R.rrl_set_profiling(tl.inst, True)
            R.rrl_reset_profile(tl.inst)
            rng = np.random.default_rng(12345)
            sets = ops = 0
            host_s = 0.0
            evs = []
            for m in range(args.moves):
                par, bl = random_move(R, n, tl.tree_parent, tl.tree_blen, rng)
                ea, eb = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                ea.record(stream)
                t0 = time.perf_counter()
                if policy == "periodic" and (m + 1) % args.period == 0:
                    tl.set_tree(par, bl, "reroot")
                    host_s += time.perf_counter() - t0
                    tl.update()
                    sets += tl.sched["set_count"]
                    ops += n - 1
                else:
                    if policy == "auto":
                        a = R.rrl_schedule_update(n, tl.tree_parent, tl.tree_blen, par, bl, True)
                        b = R.rrl_schedule_update(n, tl.tree_parent, tl.tree_blen, par, bl, False)
                        use = tl.predicted_us(a) < tl.predicted_us(b)
                    else:
                        use = policy == "partial"
                    sch = tl.update_tree(par, bl, reroot=use)
                    host_s += time.perf_counter() - t0
                    sets += sch["set_count"]
                    ops += sch["op_count"]
                eb.record(stream)
                evs.append((ea, eb))
                tl.root_loglik()
            torch.cuda.synchronize()
            span = sum(a.elapsed_time(b) for a, b in evs)
            prof = R.rrl_get_profile(tl.inst)
            final = tl.root_loglik()
            full = TreeLikelihood(n, p, 4, 4, precision=32, stream_ptr=stream.cuda_stream)
            full.set_model_params(w.model, w.rates, w.cat_weights)
            full.set_tips(w.tips)
            full.set_tree(tl.tree_parent, tl.tree_blen, "level")
            ref = full.loglik()
            full.close()
            row["policies"][policy] = {
                "updatePartials_ms": prof["partials_ms"], "update_span_ms": span, "level_sets": sets, "operations": ops,
                "host_schedule_ms": host_s * 1e3, "kernel_launches": prof["kernel_launches"],
                "final_lnL": final, "full_pass_lnL": ref, "rel_diff": abs(final - ref) / abs(ref)}
            print(kind, n, p, policy, json.dumps(row["policies"][policy]), flush=True)
            tl.close()
        base = row["policies"]["never"]["updatePartials_ms"]
        for k, v in row["policies"].items():
            v["speedup_vs_never"] = base / v["updatePartials_ms"]
        results.append(row)
    os.makedirs(os.path.dirname(args.out), exist_ok=True)
    json.dump({"runs": results}, open(args.out, "w"), indent=1)


if __name__ == "__main__":
    main()
