#!/usr/bin/env python3
"""Phase timeline of the TMA-fed tcgen05 codon kernel (K3-TC5), CTA 0 (dev tool).

Builds a trace variant of the library (-DRRL_TC5_TRACE, _lib/librrl-trace.so),
runs configs[3] (256-tip paper-random, GY94+G4) one full pass to warm up, then
re-runs the widest level set alone and prints, per phase g = (tile, category,
child) of CTA 0, the clock64 stamps of every warp role:

  P  producer issued TMA (after `empty`)     C0/C1 converter start / end
  M0/M1 MMA issue start / committed           E0 epilogue inputs ready
  Er epilogue inputs read (stage/acc freed)   E1 epilogue phase done

    RRL_LIB_PATH is set by the tool itself; run on a B200 (gpurun).
"""
import ctypes as C
import os
import subprocess
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
LIB = os.path.join(ROOT, "paper_conf_ipps_ayresc18_b200", "_lib", "librrl-trace.so")


def main():
    extra = os.environ.get("TRACE_EXTRA", "")  # e.g. "-DRRL_TC5_NLO=2" (ring-depth variants)
    env = dict(os.environ, RRL_BUILD_TAG="trace", RRL_NVCC_EXTRA=("-DRRL_TC5_TRACE " + extra).strip())
    subprocess.run([sys.executable, "-m", "paper_conf_ipps_ayresc18_b200.build"], env=env, check=True,
                   cwd=ROOT)
    os.environ["RRL_LIB_PATH"] = LIB
    from paper_conf_ipps_ayresc18_b200 import TreeLikelihood, rrl as R
    from workloads import config_workload

    p = int(sys.argv[1]) if len(sys.argv) > 1 else 10_000  # argv[2]: level set (default: widest)
    w = config_workload("c3", seed=1, p=p)
    tl = TreeLikelihood(w.n, w.p, w.s, w.c, precision=32)
    tl.set_model_params(w.model, w.rates, w.cat_weights)
    tl.set_tips(w.tips)
    tl.set_tree(w.tree.parent, w.tree.blen, "reroot")
    tl.loglik()
    widths = np.diff(tl.offsets)
    k = int(sys.argv[2]) if len(sys.argv) > 2 else int(np.argmax(widths))
    a, b = int(tl.offsets[k]), int(tl.offsets[k + 1])
    ops = tl.ops[a:b].copy()
    R.rrl_update_partials(tl.inst, ops, np.array([0, b - a], np.int32))
    R.rrl_synchronize(tl.inst)
    lib = C.CDLL(LIB)
    ev = np.zeros((18, 4096), np.int64)
    kind = np.zeros(4096, np.int32)
    assert lib.rrl_debug_tc5_trace(ev.ctypes.data_as(C.c_void_p), kind.ctypes.data_as(C.c_void_p)) == 0
    ntiles = (w.p + 127) // 128
    total = ntiles * (b - a)
    grid = min(total, 148)
    my_tiles = (total - 1) // grid + 1
    nph = my_tiles * w.c * 2
    t0 = ev[0, 0]
    names = ["P", "C0", "C1", "M0", "M1", "Er", "E1", "E0"]
    order = [0, 1, 2, 3, 4, 7, 5, 6]
    print(f"level set {k}: {b - a} ops, {ntiles} tiles/op, CTA 0 runs {my_tiles} tiles = {nph} phases")
    print("g    kind " + " ".join(f"{names[i]:>7s}" for i in order) + "   (cycles from P[0])")
    for g in range(min(nph, 64)):
        row = []
        for i in order:
            v = ev[i, g]
            row.append(f"{v - t0:7d}" if v > 0 and (i not in (3, 4) or not kind[g]) else "      -")
        print(f"{g:<4d} {'tip ' if kind[g] else 'int '} " + " ".join(row))
    te = [g for g in range(nph) if (g % (2 * w.c)) == 2 * w.c - 1]
    print("tile end (cycles): Er->exponent  ->cat0 issued  ->last cat issued  ->E1")
    for g in te[:6]:
        print(f"   g {g}: {ev[8, g] - ev[5, g]:6d} {ev[9, g] - ev[8, g]:6d} {ev[10, g] - ev[9, g]:6d} "
              f"{ev[6, g] - ev[10, g]:6d}")
    e1 = ev[6, :nph] - t0
    print(f"phase period (E1 diffs): mean {np.diff(e1).mean():.0f} cycles over {nph} phases; "
          f"last E1 at {e1[-1]} cycles")
    for lab, m in (("internal", kind[:nph] == 0), ("tip", kind[:nph] == 1)):
        idx = np.nonzero(m)[0]
        if len(idx) == 0:
            continue
        conv = ev[2, idx] - ev[1, idx]
        mma = ev[4, idx] - ev[3, idx]
        epi = ev[6, idx] - ev[7, idx]
        wait_tma = ev[1, idx] - ev[0, idx]
        print(f"{lab:8s}: TMA issue->landed(conv start) {np.median(wait_tma):.0f}  conv {np.median(conv):.0f}  "
              f"MMA issue {np.median(mma) if lab == 'internal' else 0:.0f}  epilogue {np.median(epi):.0f} (median cycles)")
    # MMA issuer: which wait released each internal phase, measured from the
    # previous internal phase's commit (M1)
    idx = [g for g in range(1, nph) if kind[g] == 0 and ev[3, g] > 0]
    prev = {}
    last = None
    for g in range(nph):
        if kind[g] == 0:
            prev[g] = last
            last = g
    rows = []
    for g in idx:
        pg = prev.get(g)
        if pg is None:
            continue
        base = ev[4, pg]
        rows.append([ev[12, g] - base, ev[13, g] - base, ev[14, g] - base, ev[15, g] - base, ev[3, g] - base,
                     ev[4, g] - ev[3, g], ev[16, g] - base])
    if rows:
        print("per internal phase (first 24): b_full a_full lo_full acc_empty start issue P_issued")
        for rr in rows[:24]:
            print("   " + " ".join(f"{x:7d}" for x in rr))
        r = np.median(np.array(rows), axis=0)
        print("MMA issuer, cycles after the previous internal phase's commit (median): "
              f"b_full {r[0]:.0f}  a_full {r[1]:.0f}  lo_full {r[2]:.0f}  acc_empty {r[3]:.0f}  start {r[4]:.0f}; "
              f"issue {r[5]:.0f}; its matrix tile was issued at {r[6]:.0f}")
    tl.close()


if __name__ == "__main__":
    main()
