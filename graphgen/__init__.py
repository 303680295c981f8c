"""Seeded synthetic-graph input generators (shared by the oracle tests and the CUDA path).

This module holds none of the triangle-counting method's arithmetic: it only
draws raw edge samples ``(src[e], dst[e])`` with Philox4x32-10, as described in
DESIGN.md ("Input recipe") and SURVEY.md §8(d).  The CPU and CUDA builds in
``libgraphgen.so`` are bit-identical.
"""
from __future__ import annotations

import ctypes
import os
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB = None

# Graph500 R-MAT/Kronecker parameters a=.57, b=.19, c=.19 (d=.05) as integer
# quadrant thresholds floor(p * 2^32).
RMAT_TA = 2448131358  # floor(0.57 * 2^32)
RMAT_TAB = 3264175144  # floor(0.76 * 2^32)
RMAT_TABC = 4080218931  # floor(0.95 * 2^32)


def _lib():
    global _LIB
    if _LIB is None:
        path = os.path.join(_HERE, "libgraphgen.so")
        if not os.path.exists(path):
            raise RuntimeError(f"{path} missing: run `make` (or __graft_entry__.build())")
        lib = ctypes.CDLL(path)
        u64, u32, i32, p = ctypes.c_uint64, ctypes.c_uint32, ctypes.c_int, ctypes.c_void_p
        lib.gg_rmat_cpu.argtypes = [u64, u32, u32, u32, u32, i32, u64, u64, p, p, i32]
        lib.gg_er_cpu.argtypes = [u64, u32, u64, u64, p, p, i32]
        lib.gg_philox_block.argtypes = [p, p, p]
        for f in ("gg_rmat_cpu", "gg_er_cpu"):
            getattr(lib, f).restype = i32
        try:
            lib.gg_rmat_cuda.argtypes = [u64, u32, u32, u32, u32, i32, u64, u64, p, p, p]
            lib.gg_er_cuda.argtypes = [u64, u32, u64, u64, p, p, p]
            lib.gg_rmat_cuda.restype = i32
            lib.gg_er_cuda.restype = i32
        except AttributeError:
            pass
        _LIB = lib
    return _LIB


def philox_block(ctr, key):
    c = np.asarray(ctr, dtype=np.uint32)
    k = np.asarray(key, dtype=np.uint32)
    out = np.zeros(4, dtype=np.uint32)
    _lib().gg_philox_block(c.ctypes.data, k.ctypes.data, out.ctypes.data)
    return out


@dataclass(frozen=True)
class GraphSpec:
    """One synthetic workload: R-MAT/Kronecker (scale, edge factor) or ER (n, M)."""

    kind: str  # "rmat" or "er"
    n: int
    samples: int
    seed: int
    scale: int = 0
    scramble: bool = True

    @property
    def name(self) -> str:
        if self.kind == "rmat":
            return f"rmat-s{self.scale}-ef{self.samples >> self.scale}"
        return f"er-n{self.n}-M{self.samples}"


def rmat_spec(scale: int, edge_factor: int, seed: int, scramble: bool = True) -> GraphSpec:
    return GraphSpec("rmat", 1 << scale, edge_factor << scale, seed, scale, scramble)


def er_spec(n: int, samples: int, seed: int) -> GraphSpec:
    return GraphSpec("er", n, samples, seed)


# BASELINE.json configs (1-based numbering as in SURVEY.md §8), seed = 20210000 + cfg.
CONFIGS = {
    1: rmat_spec(16, 16, 20210001),
    2: er_spec(1 << 22, 1 << 26, 20210002),
    3: rmat_spec(22, 16, 20210003),
    4: rmat_spec(24, 32, 20210004),
    5: rmat_spec(27, 16, 20210005),
}


def generate_cpu(spec: GraphSpec, e0: int = 0, count: int | None = None, threads: int | None = None):
    """Raw samples [e0, e0+count) as two uint32 numpy arrays (CPU generator)."""
    if count is None:
        count = spec.samples - e0
    threads = threads or min(32, os.cpu_count() or 1)
    src = np.empty(count, dtype=np.uint32)
    dst = np.empty(count, dtype=np.uint32)
    lib = _lib()
    if spec.kind == "rmat":
        rc = lib.gg_rmat_cpu(spec.seed, spec.scale, RMAT_TA, RMAT_TAB, RMAT_TABC,
                             int(spec.scramble), e0, count, src.ctypes.data, dst.ctypes.data, threads)
    else:
        rc = lib.gg_er_cpu(spec.seed, spec.n, e0, count, src.ctypes.data, dst.ctypes.data, threads)
    if rc != 0:
        raise RuntimeError(f"graphgen cpu failed rc={rc}")
    return src, dst


def generate_cuda(spec: GraphSpec, src_ptr: int, dst_ptr: int, stream_ptr: int = 0,
                  e0: int = 0, count: int | None = None) -> None:
    """Raw samples into device buffers (uint32[count] each) on `stream_ptr`."""
    if count is None:
        count = spec.samples - e0
    lib = _lib()
    if spec.kind == "rmat":
        rc = lib.gg_rmat_cuda(spec.seed, spec.scale, RMAT_TA, RMAT_TAB, RMAT_TABC,
                              int(spec.scramble), e0, count, src_ptr, dst_ptr, stream_ptr)
    else:
        rc = lib.gg_er_cuda(spec.seed, spec.n, e0, count, src_ptr, dst_ptr, stream_ptr)
    if rc != 0:
        raise RuntimeError(f"graphgen cuda failed rc={rc}")
