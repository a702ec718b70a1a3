"""Small configs for compute-sanitizer (memcheck / racecheck / synccheck): every
kernel family once, checked against the oracle (dev tool; run under gpurun).

    compute-sanitizer --tool memcheck python tools/sanitize.py
"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

from tests._util import gpu_setup, oracle_run, rel  # noqa: E402
from workloads import make_workload  # noqa: E402

CASES = [
    dict(tree_kind="pectinate", n=16, p=700, model="gtr", c=4, prec=32),        # latency K2 (smem tables)
    dict(tree_kind="pectinate", n=16, p=700, model="gtr", c=4, prec=64),        # latency K2 fp64
    dict(tree_kind="yule", n=12, p=17_000, model="gtr", c=4, prec=32),          # bulk K2
    dict(tree_kind="yule", n=12, p=17_000, model="gtr", c=4, prec=64),          # bulk K2 fp64
    dict(tree_kind="random", n=10, p=300, model="gy94", c=4, prec=32),          # K3-TT + tcgen05 K3-TC5
    dict(tree_kind="random", n=10, p=130, model="gy94", c=2, prec=64),          # K3-TT fp64 + DMMA K3-D
    dict(tree_kind="random", n=10, p=130, model="gy94", c=2, prec=64, simt=True),  # SIMT codon
]

bad = 0
for cfg in CASES:
    prec = cfg.pop("prec")
    simt = cfg.pop("simt", False)
    w = make_workload(seed=3, missing_frac=0.05, **cfg)
    for graph in (False, True):
        tl = gpu_setup(w, "reroot", prec, graph=graph, codon_simt=simt)
        got = tl.loglik()
        ora = oracle_run(w).lnl
        ok = rel(got, ora) <= (1e-10 if prec == 64 else 1e-4)
        bad += not ok
        print(cfg, prec, "graph" if graph else "eager", "ok" if ok else f"MISMATCH {got} {ora}", flush=True)
        tl.close()
print("sanitize run done, mismatches:", bad)
sys.exit(1 if bad else 0)
