"""Thin ctypes binding of libpesto.so (include/pesto.h).  Argument marshalling only: every step
of the hot path runs in the library's CUDA kernels.  PyTorch provides device memory and streams.

If libpesto.so is missing this module raises at import: there is no CPU fallback.
"""

from __future__ import annotations

import ctypes as C
import os
from typing import Optional, Sequence

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
# PESTO_LIB: an alternative in-tree build of the same library (tuning experiments, scripts/)
LIB_PATH = os.environ.get("PESTO_LIB") or os.path.join(_HERE, "libpesto.so")

OK, EINVAL, ECYCLE, ENOTTOPO, EOVERFLOW, ENOMEM, ECUDA, ENCCL, ESTATE = range(9)
INFEASIBLE = (1 << 63) - 1
KEY_INVALID = (1 << 64) - 1
ORDER_CRITICAL_PATH, ORDER_FIFO, ORDER_RANDOM = 0, 1, 2
LINKS_FCFS, LINKS_UNLIMITED = 0, 1
DISPATCH_FIXED, DISPATCH_NONDELAY = 0, 1
PLACE_SINGLE, PLACE_EXPERT, PLACE_TOPO_SPLIT, PLACE_RANDOM = 0, 1, 2, 3
KEYS_TIMED, KEYS_EVAL64, KEYS_TIMED_RAW = 0, 1, 2


class PestoError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"{_STATUS.get(status, status)}: {msg}")
        self.status = status


_STATUS = {OK: "PESTO_OK", EINVAL: "PESTO_EINVAL", ECYCLE: "PESTO_ECYCLE",
           ENOTTOPO: "PESTO_ENOTTOPO", EOVERFLOW: "PESTO_EOVERFLOW", ENOMEM: "PESTO_ENOMEM",
           ECUDA: "PESTO_ECUDA", ENCCL: "PESTO_ENCCL", ESTATE: "PESTO_ESTATE"}


class GraphDesc(C.Structure):
    _fields_ = [("n_ops", C.c_int32), ("compute_ns", C.c_void_p), ("n_edges", C.c_int64),
                ("src", C.c_void_p), ("dst", C.c_void_p), ("bytes", C.c_void_p),
                ("n_devices", C.c_int32), ("allowed", C.c_void_p), ("cuda_device", C.c_int32)]


class GraphStats(C.Structure):
    _fields_ = [("n_ops", C.c_int32), ("n_devices", C.c_int32), ("n_edges", C.c_int64),
                ("live_slots", C.c_int32), ("n_tiles", C.c_int32), ("layout_bytes", C.c_int64),
                ("max_in_degree", C.c_int32), ("max_out_degree", C.c_int32),
                ("link_classes", C.c_int32), ("time32_exact", C.c_int32)]


class Roofs(C.Structure):
    _fields_ = [("int_ops_per_s", C.c_double), ("int_chain_steps_per_s", C.c_double),
                ("l2_read_gbs", C.c_double), ("l2_rmw_gbs", C.c_double),
                ("l2_buffer_bytes", C.c_int64), ("hbm_copy_gbs", C.c_double)]


class MoveStats(C.Structure):
    _fields_ = [("candidates", C.c_int64), ("invalid", C.c_int64),
                ("identical_to_base", C.c_int64), ("distinct", C.c_int64)]


class SearchDesc(C.Structure):
    _fields_ = [("n_bases", C.c_int32), ("base_x", C.c_void_p), ("base_order", C.c_void_p),
                ("k_per_base", C.c_int64), ("mix", C.c_int32 * 4), ("seed", C.c_uint64),
                ("rank", C.c_int32), ("world", C.c_int32), ("nccl_unique_id", C.c_void_p)]


# every symbol include/pesto.h declares, with (restype, argtypes)
_VP, _I32, _I64, _U64 = C.c_void_p, C.c_int32, C.c_int64, C.c_uint64
SIGNATURES = {
    "pesto_graph_create": (_I32, [C.POINTER(GraphDesc), C.POINTER(_VP)]),
    "pesto_graph_destroy": (None, [_VP]),
    "pesto_comm_model": (_I32, [_VP, _I32, _I32, _I64, _I64]),
    "pesto_graph_set_link_model": (_I32, [_VP, _I32]),
    "pesto_graph_set_dispatch": (_I32, [_VP, _I32]),
    "pesto_graph_set_constraints": (_I32, [_VP, _VP, _VP, _VP]),
    "pesto_coarsen": (_I32, [_VP, _I32, _VP, _VP]),
    "pesto_eval_coarse_exhaustive": (_I32, [_VP, _VP, _VP, _I32, _VP, _VP, _VP, _VP]),
    "pesto_graph_stats_for": (_I32, [_VP, _VP, C.POINTER(GraphStats)]),
    "pesto_seed_order": (_I32, [_VP, _I32, _U64, _VP]),
    "pesto_seed_placement": (_I32, [_VP, _I32, _VP, _VP, _U64, _VP]),
    "pesto_eval_batch": (_I32, [_VP, _VP, _VP, _I64, _I64, _VP, _VP]),
    "pesto_eval_batch_host": (_I32, [_VP, _VP, _VP, _I64, _I64, _VP, _VP]),
    "pesto_workspace_create": (_I32, [_VP, C.POINTER(_VP)]),
    "pesto_workspace_destroy": (None, [_VP]),
    "pesto_eval_batch_host_async": (_I32, [_VP, _VP, _VP, _I64, _I64, _VP, _VP]),
    "pesto_search_create": (_I32, [_VP, C.POINTER(SearchDesc), C.POINTER(_VP)]),
    "pesto_search_set_step": (_I32, [_VP, _I64]),
    "pesto_search_step": (_I32, [_VP, _VP]),
    "pesto_search_eval": (_I32, [_VP, _VP]),
    "pesto_search_reduce": (_I32, [_VP, _VP]),
    "pesto_search_keys": (_I32, [_VP, _VP, _VP]),
    "pesto_search_set_keys": (_I32, [_VP, _VP, _VP]),
    "pesto_search_commit": (_I32, [_VP, _VP]),
    "pesto_search_candidate_keys": (_I32, [_VP, _I32, _I64, _I64, _VP, _VP]),
    "pesto_search_candidate_keys_ex": (_I32, [_VP, _I32, _I64, _I64, _VP, _I32, _VP]),
    "pesto_search_set_coarse_moves": (_I32, [_VP, _VP, _I32, _I32]),
    "pesto_search_move_stats": (_I32, [_VP, _I32, _I64, _I64, _VP]),
    "pesto_search_get": (_I32, [_VP, _I32, _VP, _VP, _VP]),
    "pesto_search_step_count": (_I64, [_VP]),
    "pesto_search_swap_stats": (_I32, [_VP, _VP, _VP]),
    "pesto_search_destroy": (None, [_VP]),
    "pesto_nccl_unique_id": (_I32, [_VP]),
    "pesto_last_error": (C.c_char_p, []),
    "pesto_status_str": (C.c_char_p, [_I32]),
    "pesto_version": (_I32, []),
    "pesto_launch_count": (_I64, []),
    "pesto_measure_roofs": (_I32, [_I32, _I32, _VP]),
}

if not os.path.exists(LIB_PATH):
    raise ImportError(f"{LIB_PATH} is missing: run __graft_entry__.build() "
                      "(python paper_conf_middleware_hafeezsg021_b200/build.py); no CPU fallback")
_L = C.CDLL(LIB_PATH)
for _name, (_res, _args) in SIGNATURES.items():
    _f = getattr(_L, _name)
    _f.restype = _res
    _f.argtypes = _args


def lib() -> C.CDLL:
    return _L


def _check(status: int):
    if status != OK:
        raise PestoError(status, (_L.pesto_last_error() or b"").decode())


def _ptr(a: np.ndarray) -> int:
    return a.ctypes.data


def _stream(stream) -> Optional[int]:
    if stream is None:
        import torch
        return torch.cuda.current_stream().cuda_stream
    return getattr(stream, "cuda_stream", stream)


def launch_count() -> int:
    return int(_L.pesto_launch_count())


def nccl_unique_id() -> bytes:
    buf = (C.c_uint8 * 128)()
    _check(_L.pesto_nccl_unique_id(buf))
    return bytes(buf)


def bits_per_op(D: int) -> int:
    return 1 if D <= 2 else (2 if D <= 4 else 4)


def pack_rows(x: np.ndarray, D: int) -> np.ndarray:
    """[count, n] device codes -> [count, stride] packed rows (b bits/op, stride % 16 == 0)."""
    x = np.ascontiguousarray(x, dtype=np.uint8)
    count, n = x.shape
    b = bits_per_op(D)
    stride = ((n * b + 7) // 8 + 15) // 16 * 16
    bits = np.zeros((count, stride * 8), dtype=np.uint8)
    for k in range(b):
        bits[:, k:n * b:b] = (x >> k) & 1
    return np.packbits(bits, axis=1, bitorder="little")


class Graph:
    """A DNN op DAG with compute times, edge tensor sizes and a comm model (pesto_graph)."""

    def __init__(self, compute_ns, src, dst, nbytes, n_devices: int, allowed=None,
                 device: int = 0):
        self.p = np.ascontiguousarray(compute_ns, dtype=np.int64)
        self.src = np.ascontiguousarray(src, dtype=np.int32)
        self.dst = np.ascontiguousarray(dst, dtype=np.int32)
        self.nbytes = np.ascontiguousarray(nbytes, dtype=np.int64)
        self.allowed = None if allowed is None else np.ascontiguousarray(allowed, dtype=np.uint8)
        self.n = int(self.p.shape[0])
        self.m = int(self.src.shape[0])
        self.D = int(n_devices)
        self.device = int(device)
        d = GraphDesc(self.n, _ptr(self.p), self.m, _ptr(self.src), _ptr(self.dst),
                      _ptr(self.nbytes), self.D,
                      None if self.allowed is None else _ptr(self.allowed), self.device)
        h = C.c_void_p()
        _check(_L.pesto_graph_create(C.byref(d), C.byref(h)))
        self._h = h

    @classmethod
    def from_arrays(cls, g, device: int = 0, comm: bool = True) -> "Graph":
        """From any object with n, p, src, dst, nbytes, D, allowed (+ beta0/beta1 [D*D])."""
        G = cls(g.p, g.src, g.dst, g.nbytes, g.D, g.allowed, device)
        if comm and getattr(g, "beta0", None) is not None:
            for a in range(g.D):
                for b in range(g.D):
                    if a != b:
                        G.comm_model(a, b, int(g.beta0[a * g.D + b]), int(g.beta1[a * g.D + b]))
        return G

    def __del__(self):
        h = getattr(self, "_h", None)
        if h and _L is not None:                      # module globals are gone at exit
            _L.pesto_graph_destroy(h)
            self._h = None

    @property
    def handle(self):
        return self._h

    def comm_model(self, src_dev: int, dst_dev: int, beta0_ns: int, beta1_fs_per_byte: int):
        _check(_L.pesto_comm_model(self._h, src_dev, dst_dev, beta0_ns, beta1_fs_per_byte))

    def set_link_model(self, model: int):
        """LINKS_FCFS (default; serial FCFS queue per directed link) or LINKS_UNLIMITED."""
        _check(_L.pesto_graph_set_link_model(self._h, model))

    def set_dispatch(self, mode: int):
        """DISPATCH_FIXED (default; pi order per device) or DISPATCH_NONDELAY (row f4(i))."""
        _check(_L.pesto_graph_set_dispatch(self._h, mode))

    def set_constraints(self, mem=None, cap=None, coloc=None):
        """Row f3: per-op footprint (None: input + output tensor bytes), per-device caps
        (None: no memory constraint), colocation group per op (-1 none; None: no colocation)."""
        arrs = [None if a is None else np.ascontiguousarray(a, dt)
                for a, dt in ((mem, np.int64), (cap, np.int64), (coloc, np.int32))]
        _check(_L.pesto_graph_set_constraints(self._h, *[None if a is None else _ptr(a)
                                                          for a in arrs]))

    def coarsen(self, target: int):
        """Row f2: PAPER.md §3.3 coarsening -> (coarse_of [n] int32, n_coarse)."""
        out = np.empty(self.n, dtype=np.int32)
        nc = C.c_int32()
        _check(_L.pesto_coarsen(self._h, target, _ptr(out), C.byref(nc)))
        return out, int(nc.value)

    def eval_coarse_exhaustive(self, order, coarse_of, n_coarse: int, stream=None):
        """Row f2: every placement of the merged vertices -> (best makespan, index, x)."""
        o = np.ascontiguousarray(order, dtype=np.int32)
        co = np.ascontiguousarray(coarse_of, dtype=np.int32)
        mk, idx = C.c_int64(), C.c_int64()
        x = np.empty(self.n, dtype=np.uint8)
        _check(_L.pesto_eval_coarse_exhaustive(self._h, _ptr(o), _ptr(co), n_coarse,
                                               C.byref(mk), C.byref(idx), _ptr(x),
                                               _stream(stream)))
        return int(mk.value), int(idx.value), x

    def stats(self, order) -> dict:
        o = np.ascontiguousarray(order, dtype=np.int32)
        st = GraphStats()
        _check(_L.pesto_graph_stats_for(self._h, _ptr(o), C.byref(st)))
        return {f: getattr(st, f) for f, _ in GraphStats._fields_}

    def seed_order(self, kind: int = ORDER_CRITICAL_PATH, seed: int = 0) -> np.ndarray:
        out = np.empty(self.n, dtype=np.int32)
        _check(_L.pesto_seed_order(self._h, kind, seed, _ptr(out)))
        return out

    def seed_placement(self, kind: int, order=None, layer=None, seed: int = 0) -> np.ndarray:
        out = np.empty(self.n, dtype=np.uint8)
        o = None if order is None else np.ascontiguousarray(order, dtype=np.int32)
        ly = None if layer is None else np.ascontiguousarray(layer, dtype=np.int32)
        _check(_L.pesto_seed_placement(self._h, kind, None if o is None else _ptr(o),
                                       None if ly is None else _ptr(ly), seed, _ptr(out)))
        return out

    def eval(self, order, rows, out=None, stream=None):
        """rows: CUDA uint8 tensor [n_cand, stride] of packed codes -> CUDA int64 makespans."""
        import torch
        o = np.ascontiguousarray(order, dtype=np.int32)
        if not rows.is_cuda or rows.dtype != torch.uint8 or rows.dim() != 2 or not rows.is_contiguous():
            raise ValueError("rows must be a contiguous 2-D CUDA uint8 tensor")
        n_cand = rows.shape[0]
        if out is None:
            out = torch.empty(n_cand, dtype=torch.int64, device=rows.device)
        _check(_L.pesto_eval_batch(self._h, _ptr(o), rows.data_ptr(), rows.shape[1], n_cand,
                                   out.data_ptr(), _stream(stream)))
        return out

    def eval_host(self, order, rows: np.ndarray, out: np.ndarray = None, stream=None):
        """Host rows (ideally pinned) -> host int64 makespans (synchronous)."""
        o = np.ascontiguousarray(order, dtype=np.int32)
        n_cand, stride = rows.shape
        if out is None:
            out = np.empty(n_cand, dtype=np.int64)
        _check(_L.pesto_eval_batch_host(self._h, _ptr(o), rows.ctypes.data, stride, n_cand,
                                        out.ctypes.data, _stream(stream)))
        return out

    def workspace(self) -> "Workspace":
        return Workspace(self)


class Workspace:
    """Private evaluation scratch (pesto_workspace) for asynchronous host-buffer batches."""

    def __init__(self, graph: Graph):
        self.graph = graph
        h = _VP()
        _check(_L.pesto_workspace_create(graph._h, C.byref(h)))
        self._h = h

    def __del__(self):
        h = getattr(self, "_h", None)
        if h:
            _L.pesto_workspace_destroy(h)
            self._h = None

    def eval_host_async(self, order, rows: np.ndarray, out: np.ndarray, stream=None):
        """Enqueue rows (pinned host) -> out (pinned host int64) on `stream`; no synchronisation:
        synchronise the stream before reading `out` or reusing `rows`."""
        o = np.ascontiguousarray(order, dtype=np.int32)
        n_cand, stride = rows.shape
        if out.shape != (n_cand,) or out.dtype != np.int64:
            raise ValueError("out must be an int64 array with one entry per row")
        _check(_L.pesto_eval_batch_host_async(self._h, _ptr(o), rows.ctypes.data, stride, n_cand,
                                              out.ctypes.data, _stream(stream)))
        return out


class Search:
    """Parallel local search from P incumbents (pesto_search)."""

    def __init__(self, graph: Graph, base_x, base_order, k_per_base: int,
                 mix: Sequence[int] = (50, 20, 20, 10), seed: int = 2021, rank: int = 0,
                 world: int = 1, nccl_id: Optional[bytes] = None):
        self.graph = graph
        self.base_x = np.ascontiguousarray(base_x, dtype=np.uint8).reshape(-1, graph.n)
        self.base_order = np.ascontiguousarray(base_order, dtype=np.int32).reshape(-1, graph.n)
        self.P = self.base_x.shape[0]
        self.K = int(k_per_base)
        self.mix, self.seed, self.rank, self.world = tuple(int(v) for v in mix), int(seed), rank, world
        self._nid = None if nccl_id is None else (C.c_uint8 * 128)(*nccl_id)
        d = SearchDesc(self.P, _ptr(self.base_x), _ptr(self.base_order), self.K,
                       (C.c_int32 * 4)(*mix), seed, rank, world,
                       None if self._nid is None else C.addressof(self._nid))
        h = C.c_void_p()
        _check(_L.pesto_search_create(graph.handle, C.byref(d), C.byref(h)))
        self._h = h

    def __del__(self):
        h = getattr(self, "_h", None)
        if h and _L is not None:
            _L.pesto_search_destroy(h)
            self._h = None

    def step(self, stream=None):
        _check(_L.pesto_search_step(self._h, _stream(stream)))

    def eval(self, stream=None):
        _check(_L.pesto_search_eval(self._h, _stream(stream)))

    def reduce(self, stream=None):
        _check(_L.pesto_search_reduce(self._h, _stream(stream)))

    def keys(self, stream=None) -> np.ndarray:
        out = np.empty(self.P, dtype=np.uint64)
        _check(_L.pesto_search_keys(self._h, _ptr(out), _stream(stream)))
        return out

    def set_keys(self, keys, stream=None):
        k = np.ascontiguousarray(keys, dtype=np.uint64)
        _check(_L.pesto_search_set_keys(self._h, _ptr(k), _stream(stream)))

    def commit(self, stream=None):
        _check(_L.pesto_search_commit(self._h, _stream(stream)))

    def set_coarse_moves(self, coarse_of, n_coarse: int, pct: int):
        """search spec S9: coarse groups move merged vertices (pesto_search_set_coarse_moves)"""
        c = np.ascontiguousarray(coarse_of, dtype=np.int32)
        if c.shape != (self.graph.n,):
            raise ValueError("coarse_of must have one entry per op")
        _check(_L.pesto_search_set_coarse_moves(self._h, c.ctypes.data, int(n_coarse), int(pct)))

    def candidate_keys(self, base: int, j0: int, j1: int, stream=None,
                       kernel: int = KEYS_TIMED) -> np.ndarray:
        """Per-candidate keys of [j0, j1) (pesto_search_candidate_keys_ex): KEYS_TIMED = the
        instantiation the step launches (exact), KEYS_EVAL64 = the independent 64-bit kernel,
        KEYS_TIMED_RAW = the timed kernel's own output (saturated walks clamped)."""
        import torch
        out = torch.empty(max(1, j1 - j0), dtype=torch.int64, device=f"cuda:{self.graph.device}")
        _check(_L.pesto_search_candidate_keys_ex(self._h, base, j0, j1, out.data_ptr(), kernel,
                                                 _stream(stream)))
        torch.cuda.synchronize(self.graph.device)
        return out[:j1 - j0].cpu().numpy().view(np.uint64)

    def move_stats(self, base: int, j0: int = 0, j1: int = None) -> dict:
        """Distinct / identical / invalid counts of the step's candidates [j0, j1) of `base`
        (pesto_search_move_stats)."""
        st = MoveStats()
        _check(_L.pesto_search_move_stats(self._h, base, j0, self.K if j1 is None else j1,
                                          C.byref(st)))
        return {f: getattr(st, f) for f, _ in MoveStats._fields_}

    def get(self, base: int):
        mk = C.c_int64()
        x = np.empty(self.graph.n, dtype=np.uint8)
        o = np.empty(self.graph.n, dtype=np.int32)
        _check(_L.pesto_search_get(self._h, base, C.byref(mk), _ptr(x), _ptr(o)))
        return int(mk.value), x, o

    @property
    def step_count(self) -> int:
        return int(_L.pesto_search_step_count(self._h))

    def set_step(self, step: int):
        _check(_L.pesto_search_set_step(self._h, int(step)))

    def checkpoint(self) -> dict:
        """Everything a resumed search needs (pesto_search_set_step): incumbents, step, K, mix,
        seed.  Save with np.savez(path, **ckpt)."""
        got = [self.get(b) for b in range(self.P)]
        return {"x": np.stack([g[1] for g in got]), "order": np.stack([g[2] for g in got]),
                "makespan": np.asarray([g[0] for g in got], np.int64),
                "step": np.int64(self.step_count), "k_per_base": np.int64(self.K),
                "mix": np.asarray(self.mix, np.int32), "seed": np.uint64(self.seed)}

    @classmethod
    def resume(cls, graph: "Graph", ckpt, rank: int = 0, world: int = 1,
               nccl_id: Optional[bytes] = None) -> "Search":
        """A search that continues a checkpoint (a dict from checkpoint() or an np.load of it)
        exactly: same incumbents, parameters and step counter."""
        S = cls(graph, ckpt["x"], ckpt["order"], int(ckpt["k_per_base"]),
                tuple(int(v) for v in ckpt["mix"]), int(ckpt["seed"]), rank, world, nccl_id)
        S.set_step(int(ckpt["step"]))
        return S

    def swap_stats(self) -> tuple:
        """(committed swaps patched in place on the device, swaps that rebuilt a layout)."""
        a, b = C.c_int64(), C.c_int64()
        _check(_L.pesto_search_swap_stats(self._h, C.byref(a), C.byref(b)))
        return int(a.value), int(b.value)


def measure_roofs(device: int = 0, reps: int = 5) -> dict:
    """SURVEY 8(d) roof microbenchmarks on `device` (pesto_measure_roofs)."""
    r = Roofs()
    _check(_L.pesto_measure_roofs(device, reps, C.byref(r)))
    return {k: getattr(r, k) for k, _ in Roofs._fields_}
