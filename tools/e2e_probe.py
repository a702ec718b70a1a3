#!/usr/bin/env python3
"""Host-side breakdown of bench.py's e2e step at configs[1] (dev probe, GPU):
wall time of each public call of one end-to-end step (set_tips from pinned
memory, set_tree with rerooting, update, root lnL to the device, D2H read),
median over steps.

    python tools/e2e_probe.py [c1] [--steps 200]
"""
import argparse
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("config", nargs="?", default="c1")
    ap.add_argument("--steps", type=int, default=200)
    a = ap.parse_args()
    import torch
    from paper_conf_ipps_ayresc18_b200 import TreeLikelihood
    from workloads import config_workload

    stream = torch.cuda.Stream()
    torch.cuda.set_stream(stream)
    w = config_workload(a.config)
    d_out = torch.zeros(1, dtype=torch.float64, device="cuda")
    tl = TreeLikelihood(w.n, w.p, w.s, w.c, precision=32, cuda_graph=True, stream_ptr=stream.cuda_stream)
    tl.set_model_params(w.model, w.rates, w.cat_weights)
    tl.set_pattern_weights(w.pattern_weights)
    pinned = torch.empty(w.tips.shape, dtype=torch.uint8, pin_memory=True).numpy()
    pinned[:] = w.tips
    names = ["set_tips", "set_tree", "update", "root", "d2h"]
    t = np.zeros((a.steps, len(names) + 1))
    for i in range(a.steps + 5):
        c0 = time.perf_counter()
        tl.set_tips(pinned)
        c1 = time.perf_counter()
        tl.set_tree(w.tree.parent, w.tree.blen, "reroot")
        c2 = time.perf_counter()
        tl.update()
        c3 = time.perf_counter()
        tl.root_loglik_device(d_out.data_ptr())
        c4 = time.perf_counter()
        float(d_out.item())
        c5 = time.perf_counter()
        if i >= 5:
            t[i - 5] = [c1 - c0, c2 - c1, c3 - c2, c4 - c3, c5 - c4, c5 - c0]
    med = np.median(t, axis=0) * 1e6
    print("median us per call: " + "  ".join(f"{n} {v:.1f}" for n, v in zip(names + ["total"], med)))
    tl.close()


if __name__ == "__main__":
    main()
