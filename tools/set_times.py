"""Per-level-set updatePartials time (dev helper, GPU): each set submitted as
its own rrl_update_partials call, bracketed by CUDA events on the instance's
stream, after a full warm pass.  Shows where a pass's time goes (wide sets vs
the latency of narrow ones).

    python tools/set_times.py [c3] [--precision 32] [--mode reroot] [--reps 20]
"""
import argparse
import json
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("config", nargs="?", default="c3")
    ap.add_argument("--precision", type=int, default=32)
    ap.add_argument("--mode", default="reroot")
    ap.add_argument("--reps", type=int, default=20)
    a = ap.parse_args()
    import torch
    from paper_conf_ipps_ayresc18_b200 import TreeLikelihood, rrl as R
    from workloads import config_workload
    torch.cuda.set_stream(torch.cuda.Stream())
    st = torch.cuda.current_stream()
    w = config_workload(a.config)
    tl = TreeLikelihood(w.n, w.p, w.s, w.c, precision=a.precision, stream_ptr=st.cuda_stream)
    tl.set_model_params(w.model, w.rates, w.cat_weights)
    tl.set_tips(w.tips)
    tl.set_pattern_weights(w.pattern_weights)
    tl.set_tree(w.tree.parent, w.tree.blen, a.mode)
    tl.update()
    ops, off = tl.ops, np.asarray(tl.offsets)
    nset = len(off) - 1
    times = np.zeros((a.reps, nset))
    for r in range(a.reps + 2):
        evs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(nset)]
        for k in range(nset):
            sub = ops[off[k]:off[k + 1]]
            evs[k][0].record(st)
            R.rrl_update_partials(tl.inst, sub, np.array([0, len(sub)], np.int32))
            evs[k][1].record(st)
        torch.cuda.synchronize()
        if r >= 2:
            times[r - 2] = [x.elapsed_time(y) * 1e3 for x, y in evs]
    med = np.median(times, axis=0)
    rows = [{"set": k, "ops": int(off[k + 1] - off[k]), "us": round(float(med[k]), 2)} for k in range(nset)]
    print(json.dumps({"config": a.config, "precision": a.precision, "mode": a.mode,
                      "total_us": round(float(med.sum()), 1), "sets": rows}))
    tl.close()


if __name__ == "__main__":
    main()
