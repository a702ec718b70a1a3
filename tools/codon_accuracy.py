#!/usr/bin/env python3
"""Accuracy of the fp32 codon kernels (dev tool, run under gpurun).

    python tools/codon_accuracy.py [--out gpurun_out/codon_accuracy.json]

For each kernel -- SIMT fp32 (RRL_FLAG_CODON_SIMT) and the tensor-core path
(K3-TT cherries + K3-TC5) --
  * one operation on controlled dense positive inputs (two internal children,
    c = 1, no rescaling): max relative error per element and the mean signed
    relative error (bias) against an fp64 evaluation of the same fp32 inputs;
  * configs[3]'s 256-tip tree rerooted (27 level sets) at 1,000 patterns:
    per-node error (reading A19 metric) against the fp64 oracle, max per
    node height;
and, as the floor any fp32 implementation has on that tree, the oracle's own
algorithm run in float32 (P rounded to fp32, numpy/BLAS sgemm, fp32
products).
"""
import argparse
import json
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

VARIANTS = ("simt", "tc5")


def one_op(R, simt, rng):
    p, s, c = 1024, 61, 1
    inst = R.rrl_create_instance(2, 5, s, p, c, 4, 1, 0, 0, 32, R.FLAG_CODON_SIMT if simt else 0)
    A1 = rng.uniform(0, 1, (c, p, s)).astype(np.float32)
    A2 = rng.uniform(0, 1, (c, p, s)).astype(np.float32)
    P1 = rng.uniform(0, 2.0 / s, (c, s, s)).astype(np.float32)
    P2 = rng.uniform(0, 2.0 / s, (c, s, s)).astype(np.float32)
    R.rrl_set_partials(inst, 2, A1.astype(np.float64))
    R.rrl_set_partials(inst, 3, A2.astype(np.float64))
    R.rrl_set_transition_matrix(inst, 0, P1.astype(np.float64))
    R.rrl_set_transition_matrix(inst, 1, P2.astype(np.float64))
    R.rrl_update_partials(inst, np.array([[4, -1, -1, 2, 0, 3, 1]], np.int32), np.array([0, 1], np.int32))
    got = R.rrl_get_partials(inst, 4, c, p, s)
    R.rrl_finalize_instance(inst)
    v1 = np.einsum("cpx,czx->cpz", A1.astype(np.float64), P1.astype(np.float64))
    v2 = np.einsum("cpx,czx->cpz", A2.astype(np.float64), P2.astype(np.float64))
    exp = v1 * v2
    r = (got - exp) / exp
    return {"max_rel": float(np.abs(r).max()), "bias_mean_rel": float(r.mean()), "rms_rel": float(np.sqrt((r * r).mean()))}


def depth_errors(simt):
    from oracle import reroot as orr
    from tests._util import gpu_setup, node_partial_error, oracle_run, rooted
    from workloads import config_workload
    w = config_workload("c3", seed=1, p=1000)
    tl = gpu_setup(w, "reroot", 32, codon_simt=simt)
    tl.update()
    rt = rooted(tl)
    ora = oracle_run(w, tree=rt, keep_partials=True)
    h = orr.heights(rt)
    by_h = {}
    for v, L in ora.partials.items():
        e = float(node_partial_error(tl.partials(v), tl.scale(v - w.n), L, ora.cum_exponent[v]).max())
        by_h[int(h[v])] = max(by_h.get(int(h[v]), 0.0), e)
    tl.close()
    return by_h, w, rt, ora


def fp32_floor(w, rt, ora):
    from oracle import model as om, pruning, reroot as orr
    from tests._util import node_partial_error
    Q = om.rate_matrix(w.model)
    ch = pruning.children_of(rt.parent)
    c, p, s = w.c, w.p, w.s
    L, E = {}, {}
    for v in range(w.n):
        L[v] = np.broadcast_to(pruning.tip_partials(w.tips[v], s).astype(np.float32), (c, p, s))
        E[v] = np.zeros(p, np.int64)
    h = orr.heights(rt)
    by_h = {}
    for v in pruning.postorder(rt.parent):
        a, b = ch[v]
        out = np.empty((c, p, s), np.float32)
        for k in range(c):
            Pa = pruning.transition_matrix(Q, w.rates[k] * rt.blen[a]).astype(np.float32)
            Pb = pruning.transition_matrix(Q, w.rates[k] * rt.blen[b]).astype(np.float32)
            out[k] = (L[a][k] @ Pa.T) * (L[b][k] @ Pb.T)
        e = np.frexp(out.max(axis=(0, 2)))[1].astype(np.int64)
        L[v] = np.ldexp(out, -e[None, :, None]).astype(np.float32)
        E[v] = E[a] + E[b] + e
        err = float(node_partial_error(L[v].astype(np.float64), E[v], ora.partials[v], ora.cum_exponent[v]).max())
        by_h[int(h[v])] = max(by_h.get(int(h[v]), 0.0), err)
    return by_h


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--out", default=os.path.join(ROOT, "gpurun_out", "codon_accuracy.json"))
    args = ap.parse_args()
    from paper_conf_ipps_ayresc18_b200 import build
    build.build()
    from paper_conf_ipps_ayresc18_b200 import rrl as R
    out = {}
    ctx = None
    for name in VARIANTS:
        simt = name == "simt"
        op = one_op(R, simt, np.random.default_rng(0))
        by_h, w, rt, ora = depth_errors(simt)
        ctx = (w, rt, ora)
        out[name] = {"one_op": op, "c3_node_error_by_height": by_h, "c3_max": max(by_h.values())}
        print(name, json.dumps(op), f"c3 max {max(by_h.values()):.3e} at h27 {by_h.get(27, 0):.3e}", flush=True)
    fl = fp32_floor(*ctx)
    out["fp32_emulation_floor"] = {"c3_node_error_by_height": fl, "c3_max": max(fl.values())}
    print("fp32 floor", f"c3 max {max(fl.values()):.3e}", flush=True)
    json.dump(out, open(args.out, "w"), indent=1)


if __name__ == "__main__":
    main()
