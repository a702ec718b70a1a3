"""Shared helpers for the GPU parity tests (tests only)."""
from __future__ import annotations

import numpy as np

from oracle import model as om, pruning
from workloads import Tree


def oracle_run(w, tree=None, keep_partials=False):
    Q = om.rate_matrix(w.model)
    return pruning.prune(tree if tree is not None else w.tree, Q, w.model.pi, w.rates,
                         w.cat_weights, w.tips, w.pattern_weights, keep_partials=keep_partials)


def gpu_setup(w, mode="reroot", precision=64, cumulative=True, graph=False, reuse=False,
              tree=None, codon_simt=False, fused=False):
    from paper_conf_ipps_ayresc18_b200 import TreeLikelihood
    t = tree if tree is not None else w.tree
    nbuf = None
    if reuse:
        from paper_conf_ipps_ayresc18_b200 import rrl as R
        nbuf = R.rrl_reroot_and_schedule(t.n, t.parent, t.blen, mode, True)["buffer_count"]
    tl = TreeLikelihood(w.n, w.p, w.s, w.c, precision=precision, cumulative_scaling=cumulative,
                        cuda_graph=graph, buffer_count=nbuf, codon_simt=codon_simt,
                        fused_pass=fused)
    tl.set_model_params(w.model, w.rates, w.cat_weights)
    tl.set_tips(w.tips)
    tl.set_pattern_weights(w.pattern_weights)
    tl.set_tree(t.parent, t.blen, mode, reuse_buffers=reuse)
    return tl


def rooted(tl) -> Tree:
    return Tree(n=tl.n, parent=tl.sched["parent"], blen=tl.sched["blen"])


def rel(a, b):
    return abs(a - b) / abs(b)


def node_partial_error(gpu_L, gpu_E, ora_L, ora_E):
    """Per (pattern): max_{c,z} |gpu - oracle| / max_{c,z} |oracle| after
    bringing both to the oracle's exponent (reading A19)."""
    shift = (gpu_E.astype(np.int64) - ora_E.astype(np.int64))[None, :, None]
    g = np.ldexp(gpu_L, shift)
    den = np.abs(ora_L).max(axis=(0, 2))
    num = np.abs(g - ora_L).max(axis=(0, 2))
    return num / den
