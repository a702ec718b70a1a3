"""Thin ctypes binding of the C ABI in include/rrl.h (argument marshalling only).

Every function here has the C name and forwards numpy arrays as plain
pointers; all computation happens in ``_lib/librrl.so`` (C++ host code and the
sm_100a kernels).  There is no Python or CPU fallback: if the shared library
is missing, importing this module raises.
"""
from __future__ import annotations

import ctypes as C
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("RRL_LIB_PATH") or os.path.join(_HERE, "_lib", "librrl.so")  # override: dev builds

if not os.path.exists(LIB_PATH):
    raise ImportError(f"{LIB_PATH} not built: run `python -m paper_conf_ipps_ayresc18_b200.build`"
                      " (there is no CPU fallback)")
_lib = C.CDLL(LIB_PATH)

SUCCESS = 0
ERROR_GENERAL = -1
ERROR_OUT_OF_MEMORY = -2
ERROR_UNIDENTIFIED_EXCEPTION = -3
ERROR_UNINITIALIZED_INSTANCE = -4
ERROR_OUT_OF_RANGE = -5
ERROR_NO_RESOURCE = -6
ERROR_NO_IMPLEMENTATION = -7
ERROR_FLOATING_POINT = -8
ERROR_INVALID_TREE = -9
ERROR_CUDA = -10
NONE = -1

FLAG_SCALE_CUMULATIVE = 0x1
FLAG_CUDA_GRAPH = 0x2
FLAG_CODON_SIMT = 0x4
FLAG_FUSED_PASS = 0x8
SCHED_SEQUENTIAL = 1
SCHED_LEVEL = 2
SCHED_REROOT = 3
SCHED_REUSE_BUFFERS = 0x100
PATTERN_RANGE_ALIGN = 512
SCHED_MODES = {"sequential": SCHED_SEQUENTIAL, "level": SCHED_LEVEL, "reroot": SCHED_REROOT}

OP_DTYPE = np.dtype([("dest", "<i4"), ("dest_scale_write", "<i4"), ("dest_scale_read", "<i4"),
                     ("child1", "<i4"), ("matrix1", "<i4"), ("child2", "<i4"), ("matrix2", "<i4")])


class rrl_profile(C.Structure):
    _fields_ = [("partials_ms", C.c_double), ("partials_launches", C.c_int64),
                ("matrices_ms", C.c_double), ("matrices_launches", C.c_int64),
                ("root_ms", C.c_double), ("root_launches", C.c_int64),
                ("scale_ms", C.c_double), ("scale_launches", C.c_int64),
                ("kernel_launches", C.c_int64), ("graph_launches", C.c_int64)]


class RRLError(RuntimeError):
    def __init__(self, code: int, where: str):
        self.code = code
        msg = _lib.rrl_last_error_message().decode()
        super().__init__(f"{where}: {_lib.rrl_error_string(code).decode()} ({code}): {msg}")


_P = C.c_void_p
_I = C.c_int
_SIGS = {
    "rrl_error_string": (C.c_char_p, [_I]),
    "rrl_last_error_message": (C.c_char_p, []),
    "rrl_version": (C.c_char_p, []),
    "rrl_create_instance": (_I, [_I] * 10 + [C.c_uint32]),
    "rrl_finalize_instance": (_I, [_I]),
    "rrl_set_stream": (_I, [_I, _P]),
    "rrl_synchronize": (_I, [_I]),
    "rrl_set_tip_states": (_I, [_I, _I, _P]),
    "rrl_set_tip_states_u8": (_I, [_I, _I, _I, _P]),
    "rrl_set_tip_partials": (_I, [_I, _I, _P]),
    "rrl_set_partials": (_I, [_I, _I, _P]),
    "rrl_get_partials": (_I, [_I, _I, _P]),
    "rrl_set_pattern_weights": (_I, [_I, _P]),
    "rrl_set_state_frequencies": (_I, [_I, _I, _P]),
    "rrl_set_category_rates": (_I, [_I, _P]),
    "rrl_set_category_weights": (_I, [_I, _I, _P]),
    "rrl_set_eigen_decomposition": (_I, [_I, _I, _P, _P, _P]),
    "rrl_update_transition_matrices": (_I, [_I, _I, _P, _P, _I]),
    "rrl_set_transition_matrix": (_I, [_I, _I, _P]),
    "rrl_get_transition_matrix": (_I, [_I, _I, _P]),
    "rrl_update_partials": (_I, [_I, _P, _I, _P, _I]),
    "rrl_accumulate_scale_factors": (_I, [_I, _P, _I, _I]),
    "rrl_reset_scale_factors": (_I, [_I, _I]),
    "rrl_get_scale_factors": (_I, [_I, _I, _P]),
    "rrl_calculate_root_log_likelihoods": (_I, [_I, _I, _I, _I, _I, _P]),
    "rrl_calculate_root_log_likelihoods_device": (_I, [_I, _I, _I, _I, _I, _P]),
    "rrl_calculate_edge_log_likelihoods": (_I, [_I] * 8 + [_P]),
    "rrl_get_site_log_likelihoods": (_I, [_I, _P]),
    "rrl_set_profiling": (_I, [_I, _I]),
    "rrl_get_profile": (_I, [_I, _P]),
    "rrl_reset_profile": (_I, [_I]),
    "rrl_reroot_and_schedule": (_I, [_I, _P, _P, C.c_uint32, _P, _P, _P, _P, _P, _P, _P]),
    "rrl_reroot_edge_table": (_I, [_I, _P, _P, _P, _P]),
    "rrl_model_eigensystem": (_I, [C.c_char_p, _I, _P, _P, _I, _P, _P, _P, _P]),
    "rrl_schedule_partial": (_I, [_I, _P, _P, _I, _P, _P, _P, _P]),
    "rrl_set_category_rates_idx": (_I, [_I, _I, _P]),
    "rrl_update_partials_ranged": (_I, [_I, _P, _P, _I, _P, _I]),
    "rrl_calculate_root_log_likelihoods_range": (_I, [_I] * 7 + [_P]),
    "rrl_reroot_exhaustive": (_I, [_I, _P, _P, _P, _P]),
    "rrl_tree_spr": (_I, [_I, _P, _P, _I, _I, _P, _P]),
    "rrl_tree_nni": (_I, [_I, _P, _P, _I, _I, _P, _P]),
    "rrl_schedule_update": (_I, [_I, _P, _P, _P, _P, C.c_uint32, _P, _P, _P, _P, _P, _P, _P]),
    "rrl_schedule_cost": (_I, [_I, _P, _I, _P, _I, _I, _I, _I, _I, C.c_double, C.c_double, C.c_double, _P]),
}
for _name, (_res, _args) in _SIGS.items():
    _f = getattr(_lib, _name)
    _f.restype = _res
    _f.argtypes = _args

EXPORTED = tuple(_SIGS)


def _ptr(a: np.ndarray | None):
    return None if a is None else a.ctypes.data


def _chk(code: int, where: str) -> int:
    if code < 0:
        raise RRLError(code, where)
    return code


def _c(a, dtype) -> np.ndarray:
    return np.ascontiguousarray(a, dtype=dtype)


def rrl_version() -> str:
    return _lib.rrl_version().decode()


def rrl_error_string(code: int) -> str:
    return _lib.rrl_error_string(code).decode()


def rrl_create_instance(tip_count, partials_buffer_count, state_count, pattern_count,
                        category_count, matrix_count, eigen_count, scale_buffer_count,
                        device=0, precision=32, flags=0) -> int:
    return _chk(_lib.rrl_create_instance(tip_count, partials_buffer_count, state_count,
                                         pattern_count, category_count, matrix_count, eigen_count,
                                         scale_buffer_count, device, precision, flags),
                "rrl_create_instance")


def rrl_finalize_instance(inst):
    return _chk(_lib.rrl_finalize_instance(inst), "rrl_finalize_instance")


def rrl_set_stream(inst, stream_ptr: int | None):
    return _chk(_lib.rrl_set_stream(inst, stream_ptr), "rrl_set_stream")


def rrl_synchronize(inst):
    return _chk(_lib.rrl_synchronize(inst), "rrl_synchronize")


def rrl_set_tip_states(inst, tip, states):
    a = _c(states, np.int32)
    return _chk(_lib.rrl_set_tip_states(inst, tip, _ptr(a)), "rrl_set_tip_states")


def rrl_set_tip_states_u8(inst, first_tip, states2d, pattern_count: int):
    """states2d: uint8 [count, pattern_count] (the C side copies rows of
    exactly pattern_count bytes, so the width is checked here)."""
    a = _c(states2d, np.uint8)
    if a.ndim != 2 or a.shape[1] != pattern_count:
        raise ValueError(f"tip states must be [count, {pattern_count}] uint8, got shape {a.shape}")
    return _chk(_lib.rrl_set_tip_states_u8(inst, first_tip, a.shape[0], _ptr(a)),
                "rrl_set_tip_states_u8")


def rrl_set_tip_partials(inst, tip, partials):
    a = _c(partials, np.float64)
    return _chk(_lib.rrl_set_tip_partials(inst, tip, _ptr(a)), "rrl_set_tip_partials")


def rrl_set_partials(inst, buffer, partials):
    a = _c(partials, np.float64)
    return _chk(_lib.rrl_set_partials(inst, buffer, _ptr(a)), "rrl_set_partials")


def rrl_get_partials(inst, buffer, c, p, s) -> np.ndarray:
    out = np.empty((c, p, s), dtype=np.float64)
    _chk(_lib.rrl_get_partials(inst, buffer, _ptr(out)), "rrl_get_partials")
    return out


def rrl_set_pattern_weights(inst, w):
    a = _c(w, np.float64)
    return _chk(_lib.rrl_set_pattern_weights(inst, _ptr(a)), "rrl_set_pattern_weights")


def rrl_set_state_frequencies(inst, idx, pi):
    a = _c(pi, np.float64)
    return _chk(_lib.rrl_set_state_frequencies(inst, idx, _ptr(a)), "rrl_set_state_frequencies")


def rrl_set_category_rates(inst, r):
    a = _c(r, np.float64)
    return _chk(_lib.rrl_set_category_rates(inst, _ptr(a)), "rrl_set_category_rates")


def rrl_set_category_weights(inst, idx, w):
    a = _c(w, np.float64)
    return _chk(_lib.rrl_set_category_weights(inst, idx, _ptr(a)), "rrl_set_category_weights")


def rrl_set_eigen_decomposition(inst, idx, V, Vinv, lam):
    V, Vi, L = _c(V, np.float64), _c(Vinv, np.float64), _c(lam, np.float64)
    return _chk(_lib.rrl_set_eigen_decomposition(inst, idx, _ptr(V), _ptr(Vi), _ptr(L)),
                "rrl_set_eigen_decomposition")


def rrl_update_transition_matrices(inst, eigen_idx, matrix_idx, t):
    mi, tt = _c(matrix_idx, np.int32), _c(t, np.float64)
    return _chk(_lib.rrl_update_transition_matrices(inst, eigen_idx, _ptr(mi), _ptr(tt), mi.shape[0]),
                "rrl_update_transition_matrices")


def rrl_set_transition_matrix(inst, idx, P):
    a = _c(P, np.float64)
    return _chk(_lib.rrl_set_transition_matrix(inst, idx, _ptr(a)), "rrl_set_transition_matrix")


def rrl_get_transition_matrix(inst, idx, c, s) -> np.ndarray:
    out = np.empty((c, s, s), dtype=np.float64)
    _chk(_lib.rrl_get_transition_matrix(inst, idx, _ptr(out)), "rrl_get_transition_matrix")
    return out


def as_ops(ops) -> np.ndarray:
    if isinstance(ops, np.ndarray) and ops.dtype == OP_DTYPE:
        return np.ascontiguousarray(ops)
    arr = np.asarray(ops, dtype=np.int32).reshape(-1, 7)
    return np.ascontiguousarray(arr).view(OP_DTYPE).reshape(-1)


def rrl_update_partials(inst, ops, set_offsets=None):
    o = as_ops(ops)
    if set_offsets is None:
        return _chk(_lib.rrl_update_partials(inst, _ptr(o), o.shape[0], None, 0), "rrl_update_partials")
    so = _c(set_offsets, np.int32)
    return _chk(_lib.rrl_update_partials(inst, _ptr(o), o.shape[0], _ptr(so), so.shape[0] - 1),
                "rrl_update_partials")


def rrl_accumulate_scale_factors(inst, scale_idx, cumulative_idx):
    a = _c(scale_idx, np.int32)
    return _chk(_lib.rrl_accumulate_scale_factors(inst, _ptr(a), a.shape[0], cumulative_idx),
                "rrl_accumulate_scale_factors")


def rrl_reset_scale_factors(inst, cumulative_idx):
    return _chk(_lib.rrl_reset_scale_factors(inst, cumulative_idx), "rrl_reset_scale_factors")


def rrl_get_scale_factors(inst, idx, p) -> np.ndarray:
    out = np.empty(p, dtype=np.int32)
    _chk(_lib.rrl_get_scale_factors(inst, idx, _ptr(out)), "rrl_get_scale_factors")
    return out


def rrl_calculate_root_log_likelihoods(inst, root_buffer, cat_weights_idx=0, freqs_idx=0,
                                       cumulative_idx=NONE, allow_nonfinite=False) -> float:
    out = np.zeros(1, dtype=np.float64)
    rc = _lib.rrl_calculate_root_log_likelihoods(inst, root_buffer, cat_weights_idx, freqs_idx,
                                                 cumulative_idx, _ptr(out))
    if not (allow_nonfinite and rc == ERROR_FLOATING_POINT):
        _chk(rc, "rrl_calculate_root_log_likelihoods")
    return float(out[0])


def rrl_calculate_root_log_likelihoods_device(inst, root_buffer, cat_weights_idx, freqs_idx,
                                              cumulative_idx, d_out_ptr: int):
    return _chk(_lib.rrl_calculate_root_log_likelihoods_device(inst, root_buffer, cat_weights_idx,
                                                               freqs_idx, cumulative_idx,
                                                               C.c_void_p(d_out_ptr)),
                "rrl_calculate_root_log_likelihoods_device")


def rrl_calculate_edge_log_likelihoods(inst, parent_buffer, child_buffer, matrix_idx,
                                       cat_weights_idx=0, freqs_idx=0, parent_scale_idx=NONE,
                                       child_scale_idx=NONE) -> float:
    out = np.zeros(1, dtype=np.float64)
    _chk(_lib.rrl_calculate_edge_log_likelihoods(inst, parent_buffer, child_buffer, matrix_idx,
                                                 cat_weights_idx, freqs_idx, parent_scale_idx,
                                                 child_scale_idx, _ptr(out)),
         "rrl_calculate_edge_log_likelihoods")
    return float(out[0])


def rrl_get_site_log_likelihoods(inst, p) -> np.ndarray:
    out = np.empty(p, dtype=np.float64)
    _chk(_lib.rrl_get_site_log_likelihoods(inst, _ptr(out)), "rrl_get_site_log_likelihoods")
    return out


def rrl_set_profiling(inst, enable: bool):
    return _chk(_lib.rrl_set_profiling(inst, 1 if enable else 0), "rrl_set_profiling")


def rrl_get_profile(inst) -> dict:
    pr = rrl_profile()
    _chk(_lib.rrl_get_profile(inst, C.addressof(pr)), "rrl_get_profile")
    return {f: getattr(pr, f) for f, _ in pr._fields_}


def rrl_reset_profile(inst):
    return _chk(_lib.rrl_reset_profile(inst), "rrl_reset_profile")


def rrl_reroot_and_schedule(tip_count, parent, blen, mode="reroot", reuse_buffers=False):
    """Returns dict(parent, blen, root_edge, ops[n-1] (OP_DTYPE), set_offsets, set_count,
    buffer_count)."""
    n = tip_count
    par = _c(parent, np.int32)
    bl = _c(blen, np.float64)
    flags = SCHED_MODES[mode] | (SCHED_REUSE_BUFFERS if reuse_buffers else 0)
    out_par = np.empty(2 * n - 1, np.int32)
    out_bl = np.empty(2 * n - 1, np.float64)
    root_edge = np.zeros(1, np.int32)
    ops = np.empty(n - 1, OP_DTYPE)
    offs = np.empty(n, np.int32)
    nsets = np.zeros(1, np.int32)
    nbuf = np.zeros(1, np.int32)
    _chk(_lib.rrl_reroot_and_schedule(n, _ptr(par), _ptr(bl), flags, _ptr(out_par), _ptr(out_bl),
                                      _ptr(root_edge), _ptr(ops), _ptr(offs), _ptr(nsets),
                                      _ptr(nbuf)), "rrl_reroot_and_schedule")
    k = int(nsets[0])
    return dict(parent=out_par, blen=out_bl, root_edge=int(root_edge[0]), ops=ops,
                set_offsets=offs[: k + 1].copy(), set_count=k, buffer_count=int(nbuf[0]))


def rrl_reroot_edge_table(tip_count, parent):
    par = _c(parent, np.int32)
    m = 2 * tip_count - 3
    key, sets, imb = (np.empty(m, np.int32) for _ in range(3))
    k = _chk(_lib.rrl_reroot_edge_table(tip_count, _ptr(par), _ptr(key), _ptr(sets), _ptr(imb)),
             "rrl_reroot_edge_table")
    return key[:k], sets[:k], imb[:k]


def rrl_model_eigensystem(model: str, pi, params=()):
    pi = _c(pi, np.float64)
    s = pi.shape[0]
    prm = _c(params if len(params) else [0.0], np.float64)
    Q, V, Vi = (np.empty((s, s)) for _ in range(3))
    lam = np.empty(s)
    _chk(_lib.rrl_model_eigensystem(model.encode(), s, _ptr(pi), _ptr(prm), len(params), _ptr(Q),
                                    _ptr(V), _ptr(Vi), _ptr(lam)), "rrl_model_eigensystem")
    return Q, V, Vi, lam


def rrl_schedule_partial(tip_count, parent, nodes):
    """Returns dict(ops (OP_DTYPE), set_offsets, op_count, set_count)."""
    par = _c(parent, np.int32)
    nd = _c(nodes, np.int32)
    ops = np.empty(max(1, tip_count - 1), OP_DTYPE)
    offs = np.empty(tip_count, np.int32)
    nop = np.zeros(1, np.int32)
    nset = np.zeros(1, np.int32)
    _chk(_lib.rrl_schedule_partial(tip_count, _ptr(par), _ptr(nd), nd.shape[0], _ptr(ops), _ptr(offs),
                                   _ptr(nop), _ptr(nset)), "rrl_schedule_partial")
    k, m = int(nset[0]), int(nop[0])
    return dict(ops=ops[:m].copy(), set_offsets=offs[: k + 1].copy(), op_count=m, set_count=k)


def rrl_reroot_exhaustive(tip_count, parent, blen=None):
    par = _c(parent, np.int32)
    bl = None if blen is None else _c(blen, np.float64)
    key = np.zeros(1, np.int32)
    sets = np.zeros(1, np.int32)
    _chk(_lib.rrl_reroot_exhaustive(tip_count, _ptr(par), _ptr(bl), _ptr(key), _ptr(sets)),
         "rrl_reroot_exhaustive")
    return int(key[0]), int(sets[0])


def rrl_set_category_rates_idx(inst, idx, r):
    a = _c(r, np.float64)
    return _chk(_lib.rrl_set_category_rates_idx(inst, idx, _ptr(a)), "rrl_set_category_rates_idx")


def rrl_update_partials_ranged(inst, ops, pattern_ranges, set_offsets=None):
    o = as_ops(ops)
    rg = _c(pattern_ranges, np.int32).reshape(-1)
    if set_offsets is None:
        return _chk(_lib.rrl_update_partials_ranged(inst, _ptr(o), _ptr(rg), o.shape[0], None, 0),
                    "rrl_update_partials_ranged")
    so = _c(set_offsets, np.int32)
    return _chk(_lib.rrl_update_partials_ranged(inst, _ptr(o), _ptr(rg), o.shape[0], _ptr(so), so.shape[0] - 1),
                "rrl_update_partials_ranged")


def rrl_calculate_root_log_likelihoods_range(inst, root_buffer, cat_weights_idx, freqs_idx, cumulative_idx,
                                             pattern_begin, pattern_end) -> float:
    out = np.zeros(1, dtype=np.float64)
    _chk(_lib.rrl_calculate_root_log_likelihoods_range(inst, root_buffer, cat_weights_idx, freqs_idx,
                                                       cumulative_idx, pattern_begin, pattern_end, _ptr(out)),
         "rrl_calculate_root_log_likelihoods_range")
    return float(out[0])


def rrl_tree_spr(tip_count, parent, blen, prune_node, regraft_node):
    """SPR move (reading A26).  Returns (parent, blen) of the new tree."""
    par, bl = _c(parent, np.int32), _c(blen, np.float64)
    op, ob = np.empty_like(par), np.empty_like(bl)
    _chk(_lib.rrl_tree_spr(tip_count, _ptr(par), _ptr(bl), int(prune_node), int(regraft_node), _ptr(op),
                           _ptr(ob)), "rrl_tree_spr")
    return op, ob


def rrl_tree_nni(tip_count, parent, blen, edge_node, which):
    """NNI move (reading A27).  Returns (parent, blen) of the new tree."""
    par, bl = _c(parent, np.int32), _c(blen, np.float64)
    op, ob = np.empty_like(par), np.empty_like(bl)
    _chk(_lib.rrl_tree_nni(tip_count, _ptr(par), _ptr(bl), int(edge_node), int(which), _ptr(op), _ptr(ob)),
         "rrl_tree_nni")
    return op, ob


def rrl_schedule_update(tip_count, stored_parent, stored_blen, parent, blen, reroot=False):
    """Partial update after any change (reading A28).  Returns dict(parent,
    blen, root_edge, ops (OP_DTYPE), set_offsets, op_count, set_count)."""
    n = tip_count
    sp, sb = _c(stored_parent, np.int32), _c(stored_blen, np.float64)
    par, bl = _c(parent, np.int32), _c(blen, np.float64)
    out_par = np.empty(2 * n - 1, np.int32)
    out_bl = np.empty(2 * n - 1, np.float64)
    key = np.zeros(1, np.int32)
    ops = np.empty(max(1, n - 1), OP_DTYPE)
    offs = np.empty(n, np.int32)
    nop = np.zeros(1, np.int32)
    nset = np.zeros(1, np.int32)
    flags = SCHED_REROOT if reroot else SCHED_LEVEL
    _chk(_lib.rrl_schedule_update(n, _ptr(sp), _ptr(sb), _ptr(par), _ptr(bl), flags, _ptr(out_par), _ptr(out_bl),
                                  _ptr(key), _ptr(ops), _ptr(offs), _ptr(nop), _ptr(nset)), "rrl_schedule_update")
    k, m = int(nset[0]), int(nop[0])
    return dict(parent=out_par, blen=out_bl, root_edge=int(key[0]), ops=ops[:m].copy(),
                set_offsets=offs[: k + 1].copy(), op_count=m, set_count=k)


def rrl_schedule_cost(tip_count, ops, set_offsets, pattern_count, state_count, category_count, precision,
                      launch_us=2.0, hbm_gbs=6000.0, l2_bytes=126e6) -> float:
    """Predicted updatePartials time (us) of a schedule (NEXT-4 cost model)."""
    o = as_ops(ops)
    so = _c(set_offsets, np.int32)
    out = np.zeros(1, np.float64)
    _chk(_lib.rrl_schedule_cost(tip_count, _ptr(o), o.shape[0], _ptr(so), so.shape[0] - 1, pattern_count,
                                state_count, category_count, precision, float(launch_us), float(hbm_gbs),
                                float(l2_bytes), _ptr(out)), "rrl_schedule_cost")
    return float(out[0])
