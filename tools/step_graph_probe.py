#!/usr/bin/env python3
"""Where the configs[1] step's time outside updatePartials goes (dev probe, GPU).

Times, with CUDA events on the launching stream and the L2 flushed before
every rep (outside the events):
  step      K1 + level sets (library graph) + K4, as bench.py's step
  sets      the level sets alone (library graph replay)
  k1, k4    each alone
  captured  the whole step (library in eager mode) captured once into one
            CUDA graph by stream capture and replayed

    python tools/step_graph_probe.py [c1] [--reps 200]
"""
import argparse
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("config", nargs="?", default="c1")
    ap.add_argument("--reps", type=int, default=200)
    a = ap.parse_args()
    import torch
    from paper_conf_ipps_ayresc18_b200 import TreeLikelihood, rrl as R
    from workloads import config_workload

    stream = torch.cuda.Stream()
    torch.cuda.set_stream(stream)
    w = config_workload(a.config)
    flush = torch.empty(512 * 1024 * 1024 // 4, dtype=torch.float32, device="cuda")
    d_out = torch.zeros(1, dtype=torch.float64, device="cuda")

    def make(graph):
        tl = TreeLikelihood(w.n, w.p, w.s, w.c, precision=32, cuda_graph=graph, stream_ptr=stream.cuda_stream)
        tl.set_model_params(w.model, w.rates, w.cat_weights)
        tl.set_tips(w.tips)
        tl.set_pattern_weights(w.pattern_weights)
        tl.set_tree(w.tree.parent, w.tree.blen, "reroot")
        return tl

    def timeit(fn):
        for _ in range(10):
            flush.zero_()
            fn()
        torch.cuda.synchronize()
        per = []
        for _ in range(a.reps):
            flush.zero_()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            fn()
            e1.record(stream)
            per.append((e0, e1))
        torch.cuda.synchronize()
        t = np.array([x.elapsed_time(y) for x, y in per]) * 1e3
        return f"median {np.median(t):8.1f} us  best {t.min():8.1f} us"

    tl = make(True)
    k1 = lambda: R.rrl_update_transition_matrices(tl.inst, 0, tl.matrix_idx, tl.t)
    sets = lambda: R.rrl_update_partials(tl.inst, tl.ops, tl.offsets)
    k4 = lambda: tl.root_loglik_device(d_out.data_ptr())

    def step():
        tl.update()
        k4()

    print("step    ", timeit(step))
    print("sets    ", timeit(sets))
    print("k1      ", timeit(k1))
    print("k4      ", timeit(k4))
    print("k1+sets ", timeit(lambda: (k1(), sets())))
    print("sets+k4 ", timeit(lambda: (sets(), k4())))
    tl.close()

    te = make(False)
    for _ in range(3):
        te.update()
        te.root_loglik_device(d_out.data_ptr())
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    try:
        with torch.cuda.graph(g, stream=stream):
            te.update()
            te.root_loglik_device(d_out.data_ptr())
        print("captured", timeit(g.replay))
    except Exception as ex:  # noqa: BLE001
        print("capture failed:", ex)
    te.close()


if __name__ == "__main__":
    main()
