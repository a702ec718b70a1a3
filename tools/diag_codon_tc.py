#!/usr/bin/env python3
"""Diagnose the accuracy of the tcgen05 codon kernel on controlled inputs (dev tool).

One operation (two internal children), no rescaling, c = 1; the expected
result is computed here in fp64 from the SAME fp32 inputs that are uploaded.
Variants: random dense inputs; inputs already exactly representable in TF32
(so 3xTF32's lo terms are zero and only accumulation error remains).
"""
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def tf32(x):
    b = np.asarray(x, np.float32).view(np.uint32) & np.uint32(0xFFFFE000)
    return b.view(np.float32)


def main():
    from paper_conf_ipps_ayresc18_b200 import build
    build.build()
    from paper_conf_ipps_ayresc18_b200 import rrl as R
    rng = np.random.default_rng(0)
    p, s, c = 512, 61, 1
    for variant in ("dense", "tf32_exact", "A_exact", "P_exact", "scaled_mix"):
        for simt in (False, True):
            flags = R.FLAG_CODON_SIMT if simt else 0
            inst = R.rrl_create_instance(2, 5, s, p, c, 4, 1, 0, 0, 32, flags)
            A1 = rng.uniform(0, 1, (c, p, s)).astype(np.float32)
            A2 = rng.uniform(0, 1, (c, p, s)).astype(np.float32)
            P1 = rng.uniform(0, 2.0 / s, (c, s, s)).astype(np.float32)
            P2 = rng.uniform(0, 2.0 / s, (c, s, s)).astype(np.float32)
            if variant == "tf32_exact":
                A1, A2, P1, P2 = tf32(A1), tf32(A2), tf32(P1), tf32(P2)
            if variant == "A_exact":
                A1, A2 = tf32(A1), tf32(A2)
            if variant == "P_exact":
                P1, P2 = tf32(P1), tf32(P2)
            if variant == "scaled_mix":
                A1 *= np.float32(10.0) ** rng.integers(-6, 1, (c, p, s)).astype(np.float32)
                P1 *= np.float32(10.0) ** rng.integers(-6, 1, (c, s, s)).astype(np.float32)
            R.rrl_set_partials(inst, 2, A1.astype(np.float64))
            R.rrl_set_partials(inst, 3, A2.astype(np.float64))
            R.rrl_set_transition_matrix(inst, 0, P1.astype(np.float64))
            R.rrl_set_transition_matrix(inst, 1, P2.astype(np.float64))
            op = np.array([[4, -1, -1, 2, 0, 3, 1]], np.int32)
            R.rrl_update_partials(inst, op, np.array([0, 1], np.int32))
            got = R.rrl_get_partials(inst, 4, c, p, s)
            v1 = np.einsum("cpx,czx->cpz", A1.astype(np.float64), P1.astype(np.float64))
            v2 = np.einsum("cpx,czx->cpz", A2.astype(np.float64), P2.astype(np.float64))
            exp = v1 * v2
            rel_el = np.abs(got - exp) / np.abs(exp)
            rel_row = (np.abs(got - exp).max(axis=2) / np.abs(exp).max(axis=2))
            print(f"{variant:11s} {'simt' if simt else 'tc  '}: max rel/elem {rel_el.max():.3e} "
                  f"median {np.median(rel_el):.3e}  max rel/row-max {rel_row.max():.3e}", flush=True)
            R.rrl_finalize_instance(inst)


if __name__ == "__main__":
    main()
