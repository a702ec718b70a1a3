"""ORACLE -- plain, slow, obviously-correct fp64 CPU reference (TEST INFRASTRUCTURE).

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s
``cpu_baseline`` / ``--impl reference`` legs may import this package.  The
product path (``paper_conf_ipps_ayresc18_b200``) never imports it and shares
no code, headers, tables or constant generators with it; the two sides share
only the seeded input generators in ``workloads/``.

Modules:
  model   -- normalised rate matrices Q (JC69, HKY, GTR, GY94)
  pruning -- expm transition matrices, Eq. (1) post-order pruning with
             power-of-two rescaling, root and edge log-likelihoods
  reroot  -- exhaustive rerooting, greedy set counting
             (PAPER.md:128), level / sequential schedules
  brute   -- brute-force summation over ancestral states (tiny trees)

Parity pins: tests/test_oracle_*.py (closed forms, brute force, invariants,
the paper's printed set counts).  Nothing here is "parity unpinned" except the
effective-GFLOPS formula, which is a reporting convention (A16).
"""
from . import brute, model, pruning, reroot  # noqa: F401
