"""Rerooted, level-batched phylogenetic partial likelihoods on B200 (sm_100a).

From-scratch implementation of the hot path of Ayres & Cummings (IPDPSW
2018): a C-ABI library (include/rrl.h, csrc/) with hand-written CUDA kernels,
bound here with ctypes (``rrl``) plus a thin host orchestrator (``engine``)
and pattern sharding across GPUs (``parallel``).  There is no CPU fallback:
importing ``rrl`` fails loudly if librrl.so is not built.

Submodules load lazily so that ``python -m paper_conf_ipps_ayresc18_b200.build``
can (re)build the library before anything opens it.
"""
import importlib

__all__ = ["rrl", "engine", "parallel", "TreeLikelihood"]


def __getattr__(name):
    if name in ("rrl", "engine", "parallel", "build"):
        return importlib.import_module(f".{name}", __name__)
    if name == "TreeLikelihood":
        return importlib.import_module(".engine", __name__).TreeLikelihood
    raise AttributeError(name)
