"""Rerooted, level-batched phylogenetic partial likelihoods on B200 (sm_100a).

From-scratch implementation of the hot path of Ayres & Cummings (IPDPSW
2018): a C-ABI library (include/rrl.h, csrc/) with hand-written CUDA kernels,
bound here with ctypes (``rrl``) plus a thin host orchestrator (``engine``).
There is no CPU fallback: importing ``rrl`` fails loudly if librrl.so is not
built.
"""
from . import rrl  # noqa: F401
from .engine import TreeLikelihood  # noqa: F401

__all__ = ["rrl", "TreeLikelihood"]
