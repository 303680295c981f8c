"""B200-native exact triangle counting (dblp/paper_conf_sigmod_hu0l21, "Accelerating
Triangle Counting on GPU").

Thin Python binding over the C-ABI of ``include/tc.h`` (``libtc_b200.so``): the
functions below only marshal arguments; every step of the path (graph build,
directing, reordering, counting) runs in the library's sm_100a kernels (the
A-order greedy, Algorithm 2, runs as host C++ inside the library).  There is no
CPU fallback: if ``libtc_b200.so`` is missing or no CUDA device is present the
calls raise.

Low-level names mirror the C-ABI (``tc_graph_from_edges``, ``tc_direct``,
``tc_reorder``, ``tc_reorder_dist``, ``tc_count``, ``tc_count_range``, ``tc_partition``,
``tc_count_dist``, ...); :class:`Graph` is a small convenience wrapper.
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
# TC_B200_LIB: an alternative build of the same library (tools/build_variant.sh experiments)
LIB_PATH = os.environ.get("TC_B200_LIB") or os.path.join(_HERE, "libtc_b200.so")

TC_OK, TC_ERR_INVALID, TC_ERR_OOM, TC_ERR_CUDA, TC_ERR_NCCL, TC_ERR_STATE = range(6)
DIRECT = {"id": 0, "degree": 1, "paper": 2}
REORDER = {"none": 0, "degree": 1, "paper": 2}
SCHEDULE = {"auto": 0, "bucketed": 1, "range": 2, "edge_aorder": 3}
_STATUS = {1: "TC_ERR_INVALID", 2: "TC_ERR_OOM", 3: "TC_ERR_CUDA", 4: "TC_ERR_NCCL", 5: "TC_ERR_STATE"}


class TCError(RuntimeError):
    def __init__(self, status, msg):
        super().__init__(f"{_STATUS.get(status, status)}: {msg}")
        self.status = status


class AOrderParams(ctypes.Structure):
    _fields_ = [("lambda_", ctypes.c_double), ("alpha", ctypes.c_double), ("beta", ctypes.c_double),
                ("bw", ctypes.c_void_p), ("bw_len", ctypes.c_uint32), ("k", ctypes.c_uint32),
                ("order", ctypes.c_int32)]


class Stats(ctypes.Structure):
    _fields_ = [(f, ctypes.c_uint64) for f in ("n", "m", "samples", "max_degree", "max_outdeg",
                                               "eq1_lo", "eq1_hi")] + [
        ("eq3", ctypes.c_int64), ("levels", ctypes.c_uint32), ("subrounds", ctypes.c_uint32),
        ("nbuckets", ctypes.c_uint32), ("direct_rule", ctypes.c_uint32),
        ("reorder_rule", ctypes.c_uint32), ("schedule", ctypes.c_uint32),
        ("triangles", ctypes.c_uint64), ("wedges", ctypes.c_uint64), ("alg_bytes", ctypes.c_uint64),
        ("ms_build", ctypes.c_double), ("ms_direct", ctypes.c_double),
        ("ms_reorder", ctypes.c_double), ("ms_count", ctypes.c_double),
        ("ms_count_kernel", ctypes.c_double), ("count_launches", ctypes.c_uint64),
        ("eq3_units", ctypes.c_int64), ("nunits", ctypes.c_uint64), ("unit_buckets", ctypes.c_uint64)]

    def as_dict(self):
        d = {f: getattr(self, f) for f, _ in self._fields_}
        d["eq1"] = (d.pop("eq1_hi") << 64) | d.pop("eq1_lo")
        return d


_LIB = None


def lib():
    """Load libtc_b200.so (fails loudly: there is no fallback path)."""
    global _LIB
    if _LIB is None:
        if not os.path.exists(LIB_PATH):
            raise RuntimeError(f"{LIB_PATH} missing: build it with `make` or __graft_entry__.build()")
        L = ctypes.CDLL(LIB_PATH, mode=ctypes.RTLD_GLOBAL)
        p, u32, u64, i32, i64 = (ctypes.c_void_p, ctypes.c_uint32, ctypes.c_uint64, ctypes.c_int,
                                 ctypes.c_int64)
        pp = ctypes.POINTER(ctypes.c_void_p)
        sig = {
            "tc_graph_from_edges": [p, p, u64, u32, i32, p, pp],
            "tc_direct": [p, i32],
            "tc_reorder": [p, i32, p],
            "tc_reorder_dist": [p, i32, p, p, i32, i32],
            "tc_set_schedule": [p, i32],
            "tc_count": [p, p, p],
            "tc_count_range": [p, u32, u32, p, p],
            "tc_count_edges": [p, p, p],
            "tc_partition": [p, u32, p],
            "tc_nccl_get_unique_id": [p],
            "tc_nccl_comm_init": [p, i32, i32, i32, pp],
            "tc_nccl_comm_destroy": [p],
            "tc_count_dist": [p, p, i32, i32, p, p],
            "tc_analyze": [p],
            "tc_get_stats": [p, p],
            "tc_export": [p, p, p, p],
            "tc_export_graph": [p, p, p],
            "tc_export_direct": [p, p, p, p],
            "tc_export_buckets": [p, p],
            "tc_export_units": [p, p, p],
            "tc_set_option": [ctypes.c_char_p, i64],
            "tc_profile_report": [ctypes.c_char_p, u64, i32],
        }
        for name, args in sig.items():
            f = getattr(L, name)
            f.argtypes = args
            f.restype = ctypes.c_int
        L.tc_graph_free.argtypes = [p]
        L.tc_graph_free.restype = None
        L.tc_last_error.restype = ctypes.c_char_p
        L.tc_version.restype = ctypes.c_char_p
        _LIB = L
    return _LIB


def _check(status):
    if status != TC_OK:
        raise TCError(status, lib().tc_last_error().decode(errors="replace"))


def _ptr(x):
    """Raw pointer of a numpy array, torch tensor, int address or None."""
    if x is None:
        return None
    if isinstance(x, int):
        return x
    if isinstance(x, np.ndarray):
        if not x.flags["C_CONTIGUOUS"]:
            raise ValueError("array must be C-contiguous")
        return x.ctypes.data
    if hasattr(x, "data_ptr"):
        if not x.is_contiguous():
            raise ValueError("tensor must be contiguous")
        return x.data_ptr()
    raise TypeError(f"unsupported buffer type {type(x)}")


def _itemsize(x):
    if isinstance(x, np.ndarray):
        return x.itemsize
    return x.element_size()


def _default_stream(device):
    try:
        import torch
        if torch.cuda.is_available():
            return torch.cuda.current_stream(device).cuda_stream
    except Exception:  # pragma: no cover - torch optional for the binding
        pass
    return None


# ------------------------------------------------------------------ C-ABI mirrors

def tc_graph_from_edges(src, dst, num_vertices, device=0, stream=None):
    if len(src) != len(dst):
        raise ValueError("src and dst differ in length")
    if len(src) and (_itemsize(src) != 4 or _itemsize(dst) != 4):
        raise TypeError("src/dst must hold 32-bit vertex ids")
    if stream is None:
        stream = _default_stream(device)
    out = ctypes.c_void_p()
    _check(lib().tc_graph_from_edges(_ptr(src) if len(src) else None, _ptr(dst) if len(dst) else None,
                                     len(src), num_vertices, device, stream, ctypes.byref(out)))
    return out.value


def tc_direct(g, rule):
    _check(lib().tc_direct(g, DIRECT[rule] if isinstance(rule, str) else rule))


def make_aorder_params(k=32, lam=9.682, alpha=0.5, beta=0.5, bw=None, order=0):
    bwa = None if bw is None else np.ascontiguousarray(bw, dtype=np.float64)
    prm = AOrderParams(lam, alpha, beta, None if bwa is None else bwa.ctypes.data,
                       0 if bwa is None else len(bwa), k, order)
    return prm, bwa  # keep bwa alive while prm is used


def tc_reorder(g, rule, params=None):
    _check(lib().tc_reorder(g, REORDER[rule] if isinstance(rule, str) else rule,
                            None if params is None else ctypes.byref(params)))


def tc_reorder_dist(g, rule, params, comm, rank, world):
    """tc_reorder on replicas: the A-order greedy on rank 0, pi broadcast over NCCL."""
    _check(lib().tc_reorder_dist(g, REORDER[rule] if isinstance(rule, str) else rule,
                                 None if params is None else ctypes.byref(params), comm, rank, world))


def tc_set_schedule(g, sched):
    _check(lib().tc_set_schedule(g, SCHEDULE[sched] if isinstance(sched, str) else sched))


def tc_count(g, per_vertex=None):
    T = ctypes.c_uint64()
    _check(lib().tc_count(g, ctypes.byref(T), _ptr(per_vertex)))
    return T.value


def tc_count_edges(g, per_edge):
    """T and the per-edge triangle counts in canonical edge order (tc_export_graph order)."""
    T = ctypes.c_uint64()
    _check(lib().tc_count_edges(g, ctypes.byref(T), _ptr(per_edge)))
    return T.value


def tc_count_range(g, u_begin, u_end, per_vertex=None):
    T = ctypes.c_uint64()
    _check(lib().tc_count_range(g, u_begin, u_end, ctypes.byref(T), _ptr(per_vertex)))
    return T.value


def tc_partition(g, world):
    b = np.zeros(world + 1, dtype=np.uint32)
    _check(lib().tc_partition(g, world, b.ctypes.data))
    return b


def tc_nccl_get_unique_id():
    buf = ctypes.create_string_buffer(128)
    _check(lib().tc_nccl_get_unique_id(buf))
    return bytes(buf.raw)


def tc_nccl_comm_init(unique_id, rank, world, device):
    buf = ctypes.create_string_buffer(bytes(unique_id), 128)
    comm = ctypes.c_void_p()
    _check(lib().tc_nccl_comm_init(buf, rank, world, device, ctypes.byref(comm)))
    return comm.value


def tc_nccl_comm_destroy(comm):
    _check(lib().tc_nccl_comm_destroy(comm))


def tc_count_dist(g, comm, rank, world, per_vertex=None):
    T = ctypes.c_uint64()
    _check(lib().tc_count_dist(g, comm, rank, world, ctypes.byref(T), _ptr(per_vertex)))
    return T.value


def tc_analyze(g):
    _check(lib().tc_analyze(g))


def tc_get_stats(g):
    s = Stats()
    _check(lib().tc_get_stats(g, ctypes.byref(s)))
    return s.as_dict()


def tc_set_option(key, value):
    _check(lib().tc_set_option(key.encode(), int(value)))


def tc_export(g, offs=None, col=None, perm=None):
    _check(lib().tc_export(g, _ptr(offs), _ptr(col), _ptr(perm)))


def tc_export_graph(g, edges=None, degree=None):
    _check(lib().tc_export_graph(g, _ptr(edges), _ptr(degree)))


def tc_export_direct(g, outdeg=None, sub=None, dsnap=None):
    _check(lib().tc_export_direct(g, _ptr(outdeg), _ptr(sub), _ptr(dsnap)))


def tc_export_buckets(g, bucket_off):
    _check(lib().tc_export_buckets(g, _ptr(bucket_off)))


def tc_export_units(g, units, unit_off):
    _check(lib().tc_export_units(g, _ptr(units), _ptr(unit_off)))


def tc_profile_report(reset=True):
    import json
    buf = ctypes.create_string_buffer(1 << 16)
    _check(lib().tc_profile_report(buf, len(buf), 1 if reset else 0))
    return json.loads(buf.value.decode())


def tc_graph_free(g):
    if g:
        lib().tc_graph_free(g)


def tc_version():
    return lib().tc_version().decode()


def tc_last_error():
    return lib().tc_last_error().decode(errors="replace")


# ------------------------------------------------------------------ convenience wrapper

class Graph:
    """Owning wrapper over a tc_graph handle."""

    def __init__(self, src, dst, num_vertices, device=0, stream=None):
        self.n = int(num_vertices)
        self.device = device
        self._h = tc_graph_from_edges(src, dst, num_vertices, device, stream)

    def __del__(self):
        self.free()

    def free(self):
        if getattr(self, "_h", None):
            tc_graph_free(self._h)
            self._h = None

    @property
    def handle(self):
        return self._h

    def direct(self, rule="degree"):
        tc_direct(self._h, rule)
        return self

    def reorder(self, rule="none", **aorder):
        prm, keep = make_aorder_params(**aorder)
        tc_reorder(self._h, rule, prm)
        del keep
        return self

    def set_schedule(self, sched):
        tc_set_schedule(self._h, sched)
        return self

    def count(self, per_vertex=False):
        if not per_vertex:
            return tc_count(self._h)
        t = np.zeros(max(self.n, 1), dtype=np.uint64)
        T = tc_count(self._h, t)
        return T, t[: self.n]

    def count_edges(self):
        """(T, support[m]): triangles per undirected edge, canonical edge order."""
        m = int(tc_get_stats(self._h)["m"])
        te = np.zeros(max(m, 1), dtype=np.uint64)
        T = tc_count_edges(self._h, te)
        return T, te[:m]

    def count_range(self, u_begin, u_end, per_vertex=False):
        if not per_vertex:
            return tc_count_range(self._h, u_begin, u_end)
        t = np.zeros(max(self.n, 1), dtype=np.uint64)
        T = tc_count_range(self._h, u_begin, u_end, t)
        return T, t[: self.n]

    def partition(self, world):
        return tc_partition(self._h, world)

    def analyze(self):
        tc_analyze(self._h)
        return self

    def stats(self):
        return tc_get_stats(self._h)

    def export(self):
        st = self.stats()
        n, m = st["n"], st["m"]
        offs = np.zeros(n + 1, dtype=np.uint64)
        col = np.zeros(max(m, 1), dtype=np.uint32)
        perm = np.zeros(max(n, 1), dtype=np.uint32)
        tc_export(self._h, offs, col, perm)
        return offs, col[:m], perm[:n]

    def export_graph(self):
        st = self.stats()
        edges = np.zeros(max(st["m"], 1), dtype=np.uint64)
        deg = np.zeros(max(self.n, 1), dtype=np.uint32)
        tc_export_graph(self._h, edges, deg)
        return edges[: st["m"]], deg[: self.n]

    def export_direct(self, internals=False):
        od = np.zeros(max(self.n, 1), dtype=np.uint32)
        sub = np.zeros(max(self.n, 1), dtype=np.uint32) if internals else None
        dsnap = np.zeros(max(self.n, 1), dtype=np.uint32) if internals else None
        tc_export_direct(self._h, od, sub, dsnap)
        if internals:
            return od[: self.n], sub[: self.n], dsnap[: self.n]
        return od[: self.n]

    def export_buckets(self):
        nb = self.stats()["nbuckets"]
        b = np.zeros(nb + 1, dtype=np.uint32)
        tc_export_buckets(self._h, b)
        return b

    def export_units(self):
        """Edge-unit A-order (schedule "edge_aorder"): (units in bucket order as
        (u << 32) | j, bucket offsets); sizes from the library's own statistics."""
        m = self.stats()["m"]
        u = np.zeros(max(m, 1), dtype=np.uint64)
        off = np.zeros(max(m, 1) + 2, dtype=np.uint32)
        tc_export_units(self._h, u, off)
        st = self.stats()
        return u[:st["nunits"]], off[:st["unit_buckets"] + 1]


def count_triangles(src, dst, num_vertices, direct="degree", reorder="none", per_vertex=False,
                    device=0, **aorder):
    """One call through the whole path: build -> direct -> reorder -> count."""
    g = Graph(src, dst, num_vertices, device)
    try:
        g.direct(direct).reorder(reorder, **aorder)
        return g.count(per_vertex)
    finally:
        g.free()
