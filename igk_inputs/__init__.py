"""Seeded synthetic inputs shared by the oracle tests and the CUDA path.

This module holds none of the method's arithmetic: it only generates
circuit-shaped graphs, initial partitions (METIS or ID blocks) and valid
modifier streams (gen.c).  The recipe is DESIGN.md section 6.
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "libigkgen.so")
_METIS = "/usr/local/cuda/lib64/libmetis_static.a"

ED, VD, VI, EI = 0, 1, 2, 3
MODE_MIX, MODE_LITERAL, MODE_ADVERSARIAL = 0, 1, 2


def build(force: bool = False) -> str:
    src = os.path.join(_HERE, "gen.c")
    if force or not os.path.exists(_SO) or os.path.getmtime(_SO) < os.path.getmtime(src):
        cmd = ["gcc", "-O2", "-fPIC", "-shared", src, "-o", _SO]
        if os.path.exists(_METIS):
            cmd.append(_METIS)
        cmd.append("-lm")
        subprocess.check_call(cmd)
    return _SO


_lib = None


def lib():
    global _lib
    if _lib is None:
        build()
        L = C.CDLL(_SO)
        P = C.c_void_p
        L.gen_graph.restype = P
        L.gen_graph.argtypes = [C.c_int64, C.c_int64, C.c_int32, C.c_double, C.c_uint64, C.c_int]
        L.gg_n.restype = C.c_int64
        L.gg_n.argtypes = [P]
        L.gg_m2.restype = C.c_int64
        L.gg_m2.argtypes = [P]
        L.gg_copy.argtypes = [P, P, P, P, P]
        L.gg_free.argtypes = [P]
        L.gen_metis.restype = C.c_int
        L.gen_metis.argtypes = [C.c_int64, P, P, P, P, C.c_int32, P, C.POINTER(C.c_int64)]
        L.gen_stream_create.restype = P
        L.gen_stream_create.argtypes = [C.c_int64, P, P, P, P, C.c_uint64, C.c_int]
        L.gen_stream_next.restype = C.c_int64
        L.gen_stream_next.argtypes = [P, C.c_int, C.c_double, C.c_int64, C.c_int64, C.c_int64, C.c_int64]
        L.gen_stream_copy.argtypes = [P, P]
        L.gen_stream_n_total.restype = C.c_int64
        L.gen_stream_n_total.argtypes = [P]
        L.gen_stream_n_active.restype = C.c_int64
        L.gen_stream_n_active.argtypes = [P]
        L.gen_stream_region_size.restype = C.c_int64
        L.gen_stream_region_size.argtypes = [P]
        L.gen_stream_n_edges.restype = C.c_int64
        L.gen_stream_n_edges.argtypes = [P]
        L.gen_stream_free.argtypes = [P]
        _lib = L
    return _lib


@dataclass
class Graph:
    xadj: np.ndarray      # int64[n+1]
    adjncy: np.ndarray    # int32[2m]
    vwgt: np.ndarray | None    # int32[n] or None (unit)
    adjwgt: np.ndarray | None  # int32[2m] or None (unit)

    @property
    def n(self) -> int:
        return len(self.xadj) - 1

    @property
    def m(self) -> int:
        return int(self.xadj[-1]) // 2


def make_graph(n: int, fmax: int, seed: int, weighted: bool = False,
               window: int = 256, p_local: float = 0.9) -> Graph:
    """Circuit-netlist-shaped graph: driver u with fanout f ~ truncated power
    law on [1, fmax] (E[f] = 2, so average degree ~4); each sink is u +- Geom
    (mean `window`) with probability p_local, else uniform."""
    L = lib()
    h = L.gen_graph(n, fmax, window, p_local, seed, int(weighted))
    try:
        m2 = L.gg_m2(h)
        xadj = np.empty(n + 1, dtype=np.int64)
        adj = np.empty(max(m2, 1), dtype=np.int32)
        vw = np.empty(max(n, 1), dtype=np.int32)
        aw = np.empty(max(m2, 1), dtype=np.int32)
        L.gg_copy(h, xadj.ctypes.data, adj.ctypes.data, vw.ctypes.data, aw.ctypes.data)
    finally:
        L.gg_free(h)
    if weighted:
        return Graph(xadj, adj[:m2], vw[:n], aw[:m2])
    return Graph(xadj, adj[:m2], None, None)


def block_partition(n: int, k: int) -> np.ndarray:
    """Contiguous ID blocks (the generator places sinks near drivers)."""
    return (np.arange(n, dtype=np.int64) * k // max(n, 1)).astype(np.int32)


def metis_partition(g: Graph, k: int) -> tuple[np.ndarray, int]:
    """METIS_PartGraphKway, default options (ufactor 30 = 3%)."""
    L = lib()
    part = np.empty(max(g.n, 1), dtype=np.int32)
    obj = C.c_int64(0)
    st = L.gen_metis(g.n, g.xadj.ctypes.data, g.adjncy.ctypes.data,
                     None if g.vwgt is None else g.vwgt.ctypes.data,
                     None if g.adjwgt is None else g.adjwgt.ctypes.data, k, part.ctypes.data, C.byref(obj))
    if st != 1:
        raise RuntimeError(f"METIS failed with status {st}")
    return part[: g.n], int(obj.value)


class Stream:
    """Seeded modifier stream; each next() is one valid batch (B, 4) int32
    = {kind, u, v, w} against the graph produced by all earlier batches."""

    def __init__(self, g: Graph, seed: int, weighted: bool = False, region0: np.ndarray | None = None):
        L = lib()
        self._keep = (g.xadj, g.adjncy, g.adjwgt)
        r0 = None if region0 is None else np.ascontiguousarray(region0, dtype=np.int32)
        self._r0 = r0
        self._free = L.gen_stream_free  # kept: module globals may be gone at interpreter exit
        self.h = L.gen_stream_create(g.n, g.xadj.ctypes.data, g.adjncy.ctypes.data,
                                     None if g.adjwgt is None else g.adjwgt.ctypes.data,
                                     None if r0 is None else r0.ctypes.data, seed, int(weighted))

    def __del__(self):
        h = getattr(self, "h", None)
        if h:
            self._free(h)
            self.h = None

    def next(self, mode: int = MODE_MIX, frac: float = 0.01, nvd: int = 0, nvi: int = 0,
             ned: int = 0, nei: int = 0) -> np.ndarray:
        L = lib()
        cnt = L.gen_stream_next(self.h, mode, frac, nvd, nvi, ned, nei)
        out = np.empty((max(cnt, 1), 4), dtype=np.int32)
        L.gen_stream_copy(self.h, out.ctypes.data)
        return out[:cnt]

    @property
    def n_total(self) -> int:
        return int(lib().gen_stream_n_total(self.h))

    @property
    def n_active(self) -> int:
        return int(lib().gen_stream_n_active(self.h))

    @property
    def n_edges(self) -> int:
        """undirected edges of the current graph (the generator's mirror)"""
        return int(lib().gen_stream_n_edges(self.h))

    @property
    def avg_degree(self) -> float:
        return 2.0 * self.n_edges / max(self.n_active, 1)

    @property
    def region_size(self) -> int:
        return int(lib().gen_stream_region_size(self.h))


# ---------------------------------------------------------------------------
# BASELINE.json configs.  Seeds: graph 0x16B00000 + #.
# ---------------------------------------------------------------------------
CONFIGS = {
    "C1": dict(n=10_000, fmax=64, k=4, eps=0.03, iters=20, mode=MODE_LITERAL,
               literal=dict(nvd=100, nvi=100, ned=200, nei=200)),
    "C2": dict(n=1_000_000, fmax=1000, k=4, eps=0.03, iters=1000, mode=MODE_MIX, frac=0.01),
    "C3": dict(n=1_000_000, fmax=1000, k=(2, 8, 32, 64), eps=0.03, iters=100, mode=MODE_MIX,
               frac=(0.001, 0.003, 0.01, 0.03, 0.10)),
    "C4": dict(n=10_000_000, fmax=10_000, k=16, eps=0.03, iters=20, mode=MODE_MIX, frac=0.05),
    "C5": dict(n=4_000_000, fmax=1000, k=8, eps=0.03, iters=21, mode=MODE_ADVERSARIAL,
               literal=dict(nvd=40_000, nvi=20_000)),
}


def graph_seed(cfg_index: int) -> int:
    return 0x16B00000 + cfg_index


def stream_seed(gseed: int) -> int:
    return (gseed ^ 0x9E3779B97F4A7C15) & 0xFFFFFFFFFFFFFFFF


def next_batch(stream: Stream, cfg: dict, frac: float | None = None) -> np.ndarray:
    mode = cfg["mode"]
    if mode == MODE_ADVERSARIAL and stream._r0 is None:
        raise ValueError("adversarial batches need the Stream built with region0 (the part-0 indicator)")
    if mode == MODE_MIX:
        return stream.next(MODE_MIX, frac if frac is not None else cfg["frac"])
    lit = cfg["literal"]
    return stream.next(mode, 0.0, lit.get("nvd", 0), lit.get("nvi", 0), lit.get("ned", 0), lit.get("nei", 0))
