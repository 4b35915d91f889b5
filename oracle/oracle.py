"""ctypes wrapper of liboracle.so -- TEST INFRASTRUCTURE ONLY.

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference leg may
import this module.  It does not import the product package and the product never imports it.
Graph arguments are duck-typed (attributes n, p, src, dst, nbytes, D, beta0, beta1, allowed),
e.g. a workloads.dag.Graph.
"""

from __future__ import annotations

import ctypes as C
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB = None

EINVAL, ECYCLE, ENOTTOPO, EOVERFLOW, ENOMEM = -1, -2, -3, -4, -5
INFEASIBLE = (1 << 63) - 1
KEY_INVALID = (1 << 64) - 1

_i32p = np.ctypeslib.ndpointer(np.int32, flags="C_CONTIGUOUS")
_i64p = np.ctypeslib.ndpointer(np.int64, flags="C_CONTIGUOUS")
_u8p = np.ctypeslib.ndpointer(np.uint8, flags="C_CONTIGUOUS")
_u64p = np.ctypeslib.ndpointer(np.uint64, flags="C_CONTIGUOUS")


def build() -> str:
    """Compile liboracle.so with the oracle's own Makefile (gcc, no CUDA)."""
    path = os.path.join(_HERE, "liboracle.so")
    src = os.path.join(_HERE, "oracle.c")
    if not os.path.exists(path) or os.path.getmtime(path) < os.path.getmtime(src):
        subprocess.run(["make", "-s", "-C", _HERE], check=True)
    return path


class _Trace(C.Structure):
    _fields_ = [("S", C.c_void_p), ("C", C.c_void_p), ("XS", C.c_void_p), ("XA", C.c_void_p)]


def lib():
    global _LIB
    if _LIB is None:
        L = C.CDLL(build())
        G = [C.c_int32, _i64p, C.c_int64, _i32p, _i32p, _i64p, C.c_int32, _i64p, _i64p,
             C.c_void_p]
        L.oracle_transfer_ns.argtypes = [C.c_int64, C.c_int64, C.c_int64]
        L.oracle_transfer_ns.restype = C.c_int64
        L.oracle_makespan.argtypes = G + [_u8p, _i32p, C.c_void_p]
        L.oracle_makespan.restype = C.c_int64
        L.oracle_longest_path.argtypes = G + [_u8p, _i32p]
        L.oracle_longest_path.restype = C.c_int64
        L.oracle_makespan_nocongest.argtypes = G + [_u8p, _i32p]
        L.oracle_makespan_nocongest.restype = C.c_int64
        L.oracle_makespan_model.argtypes = G + [_u8p, _i32p, C.c_int32, C.c_int32, C.c_void_p]
        L.oracle_makespan_model.restype = C.c_int64
        L.oracle_candidate_keys_model.argtypes = G + [C.c_int32, C.c_int32, _u8p, _i32p,
                                                      C.c_int64, C.c_int64, C.c_uint64,
                                                      C.c_uint64, _i32p, C.c_int32, C.c_int32,
                                                      C.c_int32, _u64p]
        L.oracle_candidate_keys_model.restype = C.c_int
        L.oracle_makespan_batch.argtypes = G + [C.c_int64, _u8p, _i32p, C.c_int32, C.c_int32,
                                                _i64p]
        L.oracle_makespan_batch.restype = C.c_double
        L.oracle_bruteforce.argtypes = G + [_u8p, _i32p, C.POINTER(C.c_int64)]
        L.oracle_bruteforce.restype = C.c_int64
        L.oracle_mix64.argtypes = [C.c_uint64]
        L.oracle_mix64.restype = C.c_uint64
        L.oracle_draw.argtypes = [C.c_uint64, C.c_uint64, C.c_int32, C.c_int32, C.c_int64,
                                  C.c_int32]
        L.oracle_draw.restype = C.c_uint64
        L.oracle_candidate.argtypes = [C.c_int32, C.c_int64, _i32p, _i32p, C.c_int32,
                                       C.c_void_p, C.c_int32, C.c_int32, _u8p, _i32p,
                                       C.c_int64, C.c_uint64, C.c_uint64, _i32p, _u8p, _i32p]
        L.oracle_candidate.restype = C.c_int
        L.oracle_candidate_keys.argtypes = G + [C.c_int32, C.c_int32, _u8p, _i32p, C.c_int64,
                                                C.c_int64, C.c_uint64, C.c_uint64, _i32p,
                                                C.c_int32, _u64p]
        L.oracle_candidate_keys.restype = C.c_int
        L.oracle_search_step.argtypes = G + [C.c_int32, _u8p, _i32p, _i64p, C.c_int64,
                                             C.c_uint64, C.c_uint64, _i32p, C.c_int32,
                                             C.c_int32, _u64p]
        L.oracle_search_step.restype = C.c_int
        L.oracle_set_constraints.argtypes = [C.c_int32, C.c_int64, _i32p, _i32p, _i64p,
                                             C.c_int32, C.c_void_p, C.c_void_p, C.c_void_p]
        L.oracle_set_constraints.restype = C.c_int
        L.oracle_set_coarse_moves.argtypes = [C.c_int32, _i32p, C.c_int32, C.c_int32]
        L.oracle_set_coarse_moves.restype = C.c_int
        L.oracle_clear_coarse_moves.argtypes = []
        L.oracle_clear_coarse_moves.restype = None
        L.oracle_clear_constraints.argtypes = []
        L.oracle_clear_constraints.restype = None
        L.oracle_constraints_ok.argtypes = [C.c_int32, _u8p]
        L.oracle_constraints_ok.restype = C.c_int
        _LIB = L
    return _LIB


def _g(g):
    allowed = None if g.allowed is None else np.ascontiguousarray(g.allowed, dtype=np.uint8)
    args = (int(g.n), np.ascontiguousarray(g.p, dtype=np.int64), int(len(g.src)),
            np.ascontiguousarray(g.src, dtype=np.int32), np.ascontiguousarray(g.dst, dtype=np.int32),
            np.ascontiguousarray(g.nbytes, dtype=np.int64), int(g.D),
            np.ascontiguousarray(g.beta0, dtype=np.int64),
            np.ascontiguousarray(g.beta1, dtype=np.int64),
            None if allowed is None else allowed.ctypes.data)
    return args, allowed   # keep `allowed` alive while args are in use


def transfer_ns(nbytes: int, beta0: int, beta1_fs: int) -> int:
    return int(lib().oracle_transfer_ns(nbytes, beta0, beta1_fs))


def makespan(g, x, order, trace: bool = False):
    """Event-driven simulator.  Returns the makespan (or error code / INFEASIBLE);
    with trace=True returns (makespan, dict(S, C, XS, XA))."""
    a, keep = _g(g)
    x = np.ascontiguousarray(x, dtype=np.uint8)
    order = np.ascontiguousarray(order, dtype=np.int32)
    if not trace:
        return int(lib().oracle_makespan(*a, x, order, None))
    t = {"S": np.zeros(g.n, np.int64), "C": np.zeros(g.n, np.int64),
         "XS": np.zeros(max(1, len(g.src)), np.int64), "XA": np.zeros(max(1, len(g.src)), np.int64)}
    tr = _Trace(t["S"].ctypes.data, t["C"].ctypes.data, t["XS"].ctypes.data, t["XA"].ctypes.data)
    mk = int(lib().oracle_makespan(*a, x, order, C.byref(tr)))
    t["XS"] = t["XS"][:len(g.src)]
    t["XA"] = t["XA"][:len(g.src)]
    del keep
    return mk, t


def makespan_model(g, x, order, congestion: bool = True, nondelay: bool = False,
                   trace: bool = False):
    """Event simulator under a row-f4 variant: FCFS or congestion-free links, fixed per-device
    sequences or non-delay dispatch by pi priority.  trace=True returns (makespan, trace)."""
    a, keep = _g(g)
    x = np.ascontiguousarray(x, dtype=np.uint8)
    order = np.ascontiguousarray(order, dtype=np.int32)
    if not trace:
        return int(lib().oracle_makespan_model(*a, x, order, int(congestion), int(nondelay), None))
    t = {"S": np.zeros(g.n, np.int64), "C": np.zeros(g.n, np.int64),
         "XS": np.zeros(max(1, len(g.src)), np.int64), "XA": np.zeros(max(1, len(g.src)), np.int64)}
    tr = _Trace(t["S"].ctypes.data, t["C"].ctypes.data, t["XS"].ctypes.data, t["XA"].ctypes.data)
    mk = int(lib().oracle_makespan_model(*a, x, order, int(congestion), int(nondelay),
                                         C.byref(tr)))
    t["XS"] = t["XS"][:len(g.src)]
    t["XA"] = t["XA"][:len(g.src)]
    del keep
    return mk, t


def longest_path(g, x, order) -> int:
    a, keep = _g(g)
    return int(lib().oracle_longest_path(*a, np.ascontiguousarray(x, dtype=np.uint8),
                                         np.ascontiguousarray(order, dtype=np.int32)))


class constraints:
    """Row f3 feasibility constraints (L202 memory, L175 colocation), active inside `with`.

    mem: [n] op footprints or None (= input + output tensor bytes); cap: [D] or None;
    coloc: [n] group ids (-1 none) or None."""

    def __init__(self, g, mem=None, cap=None, coloc=None):
        self.g = g
        self.arrs = [None if a is None else np.ascontiguousarray(a, dt)
                     for a, dt in ((mem, np.int64), (cap, np.int64), (coloc, np.int32))]

    def __enter__(self):
        g = self.g
        rc = lib().oracle_set_constraints(int(g.n), int(len(g.src)),
                                          np.ascontiguousarray(g.src, np.int32),
                                          np.ascontiguousarray(g.dst, np.int32),
                                          np.ascontiguousarray(g.nbytes, np.int64), int(g.D),
                                          *[None if a is None else a.ctypes.data for a in self.arrs])
        if rc != 0:
            raise ValueError(f"oracle_set_constraints: {rc}")
        return self

    def __exit__(self, *a):
        lib().oracle_clear_constraints()

    def ok(self, x) -> bool:
        return bool(lib().oracle_constraints_ok(int(self.g.n), np.ascontiguousarray(x, np.uint8)))


class coarse_moves:
    """Group moves over merged vertices (row f2, DESIGN.md §4 S9), active inside `with`."""

    def __init__(self, g, coarse_of, n_coarse, pct):
        self.g = g
        self.coarse_of = np.ascontiguousarray(coarse_of, np.int32)
        self.n_coarse, self.pct = int(n_coarse), int(pct)

    def __enter__(self):
        rc = lib().oracle_set_coarse_moves(int(self.g.n), self.coarse_of, self.n_coarse, self.pct)
        if rc != 0:
            raise ValueError(f"oracle_set_coarse_moves: {rc}")
        return self

    def __exit__(self, *a):
        lib().oracle_clear_coarse_moves()


def makespan_nocongest(g, x, order) -> int:
    a, keep = _g(g)
    return int(lib().oracle_makespan_nocongest(*a, np.ascontiguousarray(x, dtype=np.uint8),
                                               np.ascontiguousarray(order, dtype=np.int32)))


def makespan_batch(g, xs, orders, threads: int = 0):
    """xs: [count, n] uint8; orders: [n] (shared) or [count, n].  Returns (out, seconds)."""
    a, keep = _g(g)
    xs = np.ascontiguousarray(xs, dtype=np.uint8)
    orders = np.ascontiguousarray(orders, dtype=np.int32)
    per = 1 if orders.ndim == 2 else 0
    count = xs.shape[0]
    out = np.zeros(max(1, count), dtype=np.int64)
    if threads <= 0:
        threads = len(os.sched_getaffinity(0))
    secs = lib().oracle_makespan_batch(*a, count, xs, orders, per, threads, out)
    return out[:count], float(secs)


def bruteforce(g):
    """(optimum, best_x, best_order, schedules enumerated)."""
    a, keep = _g(g)
    bx = np.zeros(g.n, np.uint8)
    bo = np.zeros(g.n, np.int32)
    cnt = C.c_int64(0)
    best = int(lib().oracle_bruteforce(*a, bx, bo, C.byref(cnt)))
    return best, bx, bo, int(cnt.value)


def mix64(z: int) -> int:
    return int(lib().oracle_mix64(z))


def draw(seed, step, P, b, j, k) -> int:
    return int(lib().oracle_draw(seed, step, P, b, j, k))


def candidate(g, P, b, base_x, base_order, j, seed, step, mix):
    """Decode candidate j of base b -> (valid, x, order).  base_x [P, n], base_order [P, n]."""
    allowed = None if g.allowed is None else np.ascontiguousarray(g.allowed, dtype=np.uint8)
    x = np.zeros(g.n, np.uint8)
    o = np.zeros(g.n, np.int32)
    ok = lib().oracle_candidate(int(g.n), int(len(g.src)), np.ascontiguousarray(g.src, np.int32),
                                np.ascontiguousarray(g.dst, np.int32), int(g.D),
                                None if allowed is None else allowed.ctypes.data, P, b,
                                np.ascontiguousarray(base_x, np.uint8),
                                np.ascontiguousarray(base_order, np.int32), j, seed, step,
                                np.asarray(mix, np.int32), x, o)
    return bool(ok), x, o


def candidate_keys(g, P, b, base_x, base_order, j0, j1, seed, step, mix, threads: int = 0):
    a, keep = _g(g)
    out = np.zeros(max(1, j1 - j0), np.uint64)
    if threads <= 0:
        threads = len(os.sched_getaffinity(0))
    rc = lib().oracle_candidate_keys(*a, P, b, np.ascontiguousarray(base_x, np.uint8),
                                     np.ascontiguousarray(base_order, np.int32), j0, j1, seed,
                                     step, np.asarray(mix, np.int32), threads, out)
    if rc != 0:
        raise ValueError(f"oracle_candidate_keys: {rc}")
    return out[:j1 - j0]


def candidate_keys_model(g, P, b, base_x, base_order, j0, j1, seed, step, mix,
                         congestion: bool = True, nondelay: bool = False, threads: int = 0):
    a, keep = _g(g)
    out = np.zeros(max(1, j1 - j0), np.uint64)
    if threads <= 0:
        threads = len(os.sched_getaffinity(0))
    rc = lib().oracle_candidate_keys_model(*a, P, b, np.ascontiguousarray(base_x, np.uint8),
                                           np.ascontiguousarray(base_order, np.int32), j0, j1,
                                           seed, step, np.asarray(mix, np.int32),
                                           int(congestion), int(nondelay), threads, out)
    if rc != 0:
        raise ValueError(f"oracle_candidate_keys_model: {rc}")
    return out[:j1 - j0]


def search_step(g, base_x, base_order, base_mk, K, seed, step, mix, world=1, threads=0):
    """In-place reference step over P bases; returns keys [P] (uint64)."""
    a, keep = _g(g)
    P = base_x.shape[0]
    keys = np.zeros(P, np.uint64)
    if threads <= 0:
        threads = len(os.sched_getaffinity(0))
    rc = lib().oracle_search_step(*a, P, base_x, base_order, base_mk, K, seed, step,
                                  np.asarray(mix, np.int32), world, threads, keys)
    if rc != 0:
        raise ValueError(f"oracle_search_step: {rc}")
    return keys
