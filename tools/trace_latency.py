#!/usr/bin/env python3
"""Per-level-set timeline of the latency-path K2 (k_partials_nuc), dev tool.

Builds a trace variant of the library (-DRRL_LAT_TRACE, _lib/librrl-lattrace.so):
every CTA stamps %globaltimer at entry, after griddepcontrol.wait and at its
end (thread 0, after its stores are issued; the record slot is claimed at entry).  Runs configs[1] (or another config) as
the bench does (CUDA graph, PDL, L2 flushed before every pass) and prints,
per level set, where the time goes:

  body     last CTA end - first CTA past its wait      (the set's own work)
  release  first CTA past the wait of set k+1 - last CTA end of set k
  skew     last CTA past the wait - first CTA past the wait
  lead     first CTA past the wait - first CTA entry   (prologue overlap)

    python tools/trace_latency.py [c1] [--mode reroot] [--passes 5]
    TRACE_EXTRA="-DRRL_LAT_THREADS=256" python tools/trace_latency.py   (variants)
"""
import argparse
import ctypes as C
import os
import subprocess
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("config", nargs="?", default="c1")
    ap.add_argument("--mode", default="reroot")
    ap.add_argument("--passes", type=int, default=5)
    ap.add_argument("--precision", type=int, default=32)
    ap.add_argument("--tag", default="lattrace")
    ap.add_argument("--no-build", action="store_true")
    ap.add_argument("--no-flush", action="store_true", help="keep L2 (and TLBs) warm between passes")
    a = ap.parse_args()
    lib_path = os.path.join(ROOT, "paper_conf_ipps_ayresc18_b200", "_lib", f"librrl-{a.tag}.so")
    if not a.no_build:
        extra = os.environ.get("TRACE_EXTRA", "")
        env = dict(os.environ, RRL_BUILD_TAG=a.tag, RRL_NVCC_EXTRA=("-DRRL_LAT_TRACE " + extra).strip())
        subprocess.run([sys.executable, "-m", "paper_conf_ipps_ayresc18_b200.build"], env=env, check=True,
                       cwd=ROOT)
    os.environ["RRL_LIB_PATH"] = lib_path
    import torch
    from paper_conf_ipps_ayresc18_b200 import TreeLikelihood
    from workloads import config_workload

    torch.cuda.set_stream(torch.cuda.Stream())
    st = torch.cuda.current_stream()
    w = config_workload(a.config)
    tl = TreeLikelihood(w.n, w.p, w.s, w.c, precision=a.precision, cuda_graph=True, stream_ptr=st.cuda_stream)
    tl.set_model_params(w.model, w.rates, w.cat_weights)
    tl.set_tips(w.tips)
    tl.set_pattern_weights(w.pattern_weights)
    tl.set_tree(w.tree.parent, w.tree.blen, a.mode)
    lib = C.CDLL(lib_path)
    rec = np.zeros((160 * 1024, 4), np.uint64)
    cnt = np.zeros(160, np.uint32)

    def read():
        assert lib.rrl_debug_lat_trace(rec.ctypes.data_as(C.c_void_p), cnt.ctypes.data_as(C.c_void_p)) == 0
        return np.concatenate([rec[s * 1024:s * 1024 + min(int(cnt[s]), 1024)] for s in range(160)])
    flush = torch.empty(512 * 1024 * 1024 // 4, dtype=torch.float32, device="cuda")
    for _ in range(5):
        tl.update()
    torch.cuda.synchronize()
    read()
    nset = len(tl.offsets) - 1
    per = []
    for _ in range(a.passes):
        if not a.no_flush:
            flush.zero_()
        tl.update()
        torch.cuda.synchronize()
        r = read()
        key = r[:, 0]
        t_entry = r[:, 2].astype(np.int64)
        d = r[:, 3]
        M = np.uint64((1 << 21) - 1)
        t_wait = t_entry + (d & M).astype(np.int64)
        d_ld = ((d >> np.uint64(21)) & M).astype(np.int64)
        t_ld = np.where(d_ld > 0, t_entry + d_ld, t_wait)
        t_end = t_entry + (d >> np.uint64(42)).astype(np.int64)
        sets = []
        for k in np.unique(key):
            m = key == k
            sets.append((t_wait[m].min(), t_wait[m].max(), t_end[m].max(), t_entry[m].min(), int(m.sum()),
                         int(np.median(t_ld[m] - t_wait[m])), int(np.max(t_ld[m]) - t_wait[m].min()),
                         int(np.median(t_end[m] - t_ld[m]))))
        sets.sort()
        per.append(np.array(sets, np.int64))
    print(f"{a.config} {a.mode} fp{a.precision}: {nset} level sets, {per[0].shape[0]} traced, "
          f"CTAs per set {np.median(per[0][:, 4]):.0f}")
    body, rel, skew, lead, span, ld, ldmax, tail = [], [], [], [], [], [], [], []
    for s in per:
        ld.append(s[:, 5])
        ldmax.append(s[:, 6])
        tail.append(s[:, 7])
        body.append(s[:, 2] - s[:, 0])
        skew.append(s[:, 1] - s[:, 0])
        lead.append(s[:, 0] - s[:, 3])
        rel.append(s[1:, 0] - s[:-1, 2])
        span.append((s[-1, 2] - s[0, 0]) / 1e3)
    body, skew, lead, rel, ld, ldmax, tail = (np.concatenate(x) for x in (body, skew, lead, rel, ld, ldmax, tail))
    q = lambda x: f"median {np.median(x):7.0f}  p10 {np.percentile(x, 10):7.0f}  p90 {np.percentile(x, 90):7.0f} ns"
    print(f"  body    {q(body)}")
    print(f"  release {q(rel)}")
    print(f"  skew    {q(skew)}")
    print(f"  lead    {q(lead)}")
    print(f"  CTA wait->loads landed (median CTA) {q(ld)}")
    print(f"  first wait->last CTA loads landed   {q(ldmax)}")
    print(f"  CTA loads landed->CTA end (median)  {q(tail)}")
    print(f"  first wait -> last end of the pass: {np.median(span):.1f} us "
          f"({np.median(span) * 1e3 / max(nset, 1):.0f} ns per set)")
    s = per[-1]
    print("  set  ctas  lead  skew  body  ld_med ld_max tail_med release(next)")
    for i in range(min(len(s), 12)):
        nx = s[i + 1, 0] - s[i, 2] if i + 1 < len(s) else 0
        print(f"  {i:3d} {s[i, 4]:5d} {s[i, 0] - s[i, 3]:5d} {s[i, 1] - s[i, 0]:5d} {s[i, 2] - s[i, 0]:5d} "
              f"{s[i, 5]:6d} {s[i, 6]:6d} {s[i, 7]:6d} {nx:6d}")
    tl.close()


if __name__ == "__main__":
    main()
