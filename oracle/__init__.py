"""ctypes wrapper of the CPU oracle (oracle/igk_oracle.c).

TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and the
cpu_baseline / --impl reference legs of bench.py may import this module.
The product package (paper_conf_dac_leejlczcshh25_b200) never imports it.
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "libigk_oracle.so")

STATS = ["affected", "inserted", "expanded", "filtered_in", "expanded_in",
         "evicted", "rounds", "moves_applied", "moves_deferred", "cut", "cap",
         "max_part_weight", "imbalanced"]

OK, EINVAL, ENOMEM, WIMBALANCED = 0, 1, 2, 6


def build(force: bool = False) -> str:
    srcs = [os.path.join(_HERE, f) for f in ("igk_oracle.c", "igk_fgp.c", "igk_oracle.h")]
    if force or not os.path.exists(_SO) or any(os.path.getmtime(_SO) < os.path.getmtime(f) for f in srcs):
        subprocess.check_call(["gcc", "-O2", "-Wall", "-fPIC", "-shared", *srcs[:2], "-o", _SO])
    return _SO


_lib = None


def lib():
    global _lib
    if _lib is None:
        build()
        L = C.CDLL(_SO)
        P = C.c_void_p
        i64p = C.POINTER(C.c_int64)
        i32p = C.POINTER(C.c_int32)
        L.ora_create.restype = P
        L.ora_create.argtypes = [C.c_int64, i64p, i32p, i32p, i32p, C.c_int32, C.c_double, i32p, C.POINTER(C.c_int)]
        L.ora_destroy.argtypes = [P]
        L.ora_last_error.restype = C.c_char_p
        L.ora_last_error.argtypes = [P]
        L.ora_apply.argtypes = [P, i32p, C.c_int64, i64p, i64p]
        L.ora_refine.argtypes = [P, i64p]
        L.ora_refine_global.argtypes = [P, i64p]
        L.ora_n_total.restype = C.c_int64
        L.ora_n_total.argtypes = [P]
        L.ora_n_active.restype = C.c_int64
        L.ora_n_active.argtypes = [P]
        L.ora_partition.argtypes = [P, i32p]
        L.ora_cut.restype = C.c_int64
        L.ora_cut.argtypes = [P]
        L.ora_part_weights.argtypes = [P, i64p]
        L.ora_total_weight.restype = C.c_int64
        L.ora_total_weight.argtypes = [P]
        L.ora_cap_value.restype = C.c_int64
        L.ora_cap_value.argtypes = [P]
        L.ora_num_slots.restype = C.c_int64
        L.ora_num_slots.argtypes = [P]
        L.ora_export_csr.argtypes = [P, i64p, i32p, i32p]
        L.ora_check_invariants.argtypes = [P, C.c_char_p, C.c_int]
        L.ora_check_invariants_ext.argtypes = [P, C.c_int64, C.c_int, C.c_char_p, C.c_int]
        L.ora_debug_set_part.argtypes = [P, C.c_int64, C.c_int32]
        L.ora_debug_set_part_weight.argtypes = [P, C.c_int32, C.c_int64]
        L.ora_debug_set_total_weight.argtypes = [P, C.c_int64]
        L.ora_debug_set_frontier.argtypes = [P, C.c_int64, C.c_int]
        L.ora_debug_add_half_edge.argtypes = [P, C.c_int64, C.c_int32, C.c_int32]
        L.ora_debug_set_edge_weight.argtypes = [P, C.c_int64, C.c_int32, C.c_int32]
        L.ora_cap.restype = C.c_int64
        L.ora_cap.argtypes = [C.c_int64, C.c_double, C.c_int32]
        L.ora_trace_rounds.restype = C.c_int64
        L.ora_trace_rounds.argtypes = [P, i64p, i64p, C.c_int64]
        L.ora_trace_moves.restype = C.c_int64
        L.ora_trace_moves.argtypes = [P, i64p, C.c_int64]
        L.ora_trace_sets.argtypes = [P, C.c_void_p, C.c_void_p, C.c_void_p]
        L.ora_fgp.restype = C.c_int
        L.ora_fgp.argtypes = [C.c_int64, i64p, i32p, i32p, i32p, C.c_int32, C.c_double, C.c_int32, i32p, i64p,
                              C.c_int64]
        L.ora_fgp_coarsen_step.restype = C.c_int64
        L.ora_fgp_coarsen_step.argtypes = [C.c_int64, i64p, i32p, i32p, C.c_int32, i32p, i32p, i32p, i32p,
                                           C.POINTER(C.c_int64)]
        L.ora_fgp_set_passes.argtypes = [C.c_int]
        L.ora_fgp_set_init.argtypes = [C.c_int]
        L.ora_fgp_set_lp_passes.argtypes = [C.c_int]
        L.ora_repartition.restype = C.c_int
        L.ora_repartition.argtypes = [P, C.c_int32]
        L.ora_fgp_lp_pass.restype = C.c_int64
        L.ora_fgp_lp_pass.argtypes = [C.c_int64, i64p, i32p, i32p, i32p, C.c_int32, C.c_double, i32p,
                                      C.POINTER(C.c_int64)]
        _lib = L
    return _lib


def _p(a, ct):
    return None if a is None else a.ctypes.data_as(C.POINTER(ct))


def fgp(xadj, adjncy, k, eps, vwgt=None, adjwgt=None, group_size=6):
    """IGK-FGP v1 full partition (NEXT-2).  Returns (part, [n per level])."""
    xadj = np.ascontiguousarray(xadj, dtype=np.int64)
    adjncy = np.ascontiguousarray(adjncy, dtype=np.int32)
    vwgt = None if vwgt is None else np.ascontiguousarray(vwgt, dtype=np.int32)
    adjwgt = None if adjwgt is None else np.ascontiguousarray(adjwgt, dtype=np.int32)
    n = len(xadj) - 1
    part = np.zeros(max(n, 1), np.int32)
    lv = np.zeros(40, np.int64)
    r = lib().ora_fgp(n, _p(xadj, C.c_int64), _p(adjncy, C.c_int32), _p(vwgt, C.c_int32), _p(adjwgt, C.c_int32),
                      k, eps, group_size, _p(part, C.c_int32), _p(lv, C.c_int64), 40)
    if r < 1:
        raise ValueError(f"ora_fgp failed ({r})")
    return part[:n], lv[:r].tolist()


def fgp_set_passes(passes: int) -> None:
    """test-only: refinement passes per FGP level (default 8)"""
    lib().ora_fgp_set_passes(passes)


def fgp_set_init(mode: int) -> None:
    """test-only: FGP initial partition, 0 = BFS growing (default), 1 = ID blocks"""
    lib().ora_fgp_set_init(mode)


def fgp_set_lp_passes(passes: int) -> None:
    """test-only: label-propagation passes per finer FGP level (default 16)"""
    lib().ora_fgp_set_lp_passes(passes)


def fgp_lp_pass(xadj, adjncy, k, eps, part, vwgt=None, adjwgt=None):
    """one label-propagation pass (reading F7): (new part, moved, cut reduction)"""
    xadj = np.ascontiguousarray(xadj, dtype=np.int64)
    adjncy = np.ascontiguousarray(adjncy, dtype=np.int32)
    vwgt = None if vwgt is None else np.ascontiguousarray(vwgt, dtype=np.int32)
    adjwgt = None if adjwgt is None else np.ascontiguousarray(adjwgt, dtype=np.int32)
    part = np.array(part, dtype=np.int32)
    dc = C.c_int64(0)
    mv = lib().ora_fgp_lp_pass(len(xadj) - 1, _p(xadj, C.c_int64), _p(adjncy, C.c_int32), _p(vwgt, C.c_int32),
                               _p(adjwgt, C.c_int32), k, eps, _p(part, C.c_int32), C.byref(dc))
    return part, int(mv), int(dc.value)


def fgp_coarsen_step(xadj, adjncy, adjwgt=None, group_size=6):
    """one coarsening step: (sel, root, label, cmap, n_groups, coarsenable)"""
    xadj = np.ascontiguousarray(xadj, dtype=np.int64)
    adjncy = np.ascontiguousarray(adjncy, dtype=np.int32)
    adjwgt = None if adjwgt is None else np.ascontiguousarray(adjwgt, dtype=np.int32)
    n = len(xadj) - 1
    out = [np.zeros(max(n, 1), np.int32) for _ in range(4)]
    co = C.c_int64(0)
    ng = lib().ora_fgp_coarsen_step(n, _p(xadj, C.c_int64), _p(adjncy, C.c_int32), _p(adjwgt, C.c_int32),
                                    group_size, *[_p(a, C.c_int32) for a in out], C.byref(co))
    return tuple(a[:n] for a in out) + (int(ng), int(co.value))


def cap(W: int, eps: float, k: int) -> int:
    return int(lib().ora_cap(W, eps, k))


class Oracle:
    """One oracle graph (IGK-SEM v1)."""

    def __init__(self, xadj, adjncy, k, eps, part, vwgt=None, adjwgt=None):
        L = lib()
        xadj = np.ascontiguousarray(xadj, dtype=np.int64)
        adjncy = np.ascontiguousarray(adjncy, dtype=np.int32)
        part = np.ascontiguousarray(part, dtype=np.int32)
        vwgt = None if vwgt is None else np.ascontiguousarray(vwgt, dtype=np.int32)
        adjwgt = None if adjwgt is None else np.ascontiguousarray(adjwgt, dtype=np.int32)
        st = C.c_int(0)
        n = len(xadj) - 1
        self.k = int(k)
        self.h = L.ora_create(n, _p(xadj, C.c_int64), _p(adjncy, C.c_int32), _p(vwgt, C.c_int32),
                              _p(adjwgt, C.c_int32), k, eps, _p(part, C.c_int32), C.byref(st))
        if not self.h:
            raise ValueError(f"ora_create rejected the input (status {st.value})")
        self._destroy = L.ora_destroy  # kept: module globals may be gone at interpreter exit

    def __del__(self):
        h = getattr(self, "h", None)
        if h:
            self._destroy(h)
            self.h = None

    def apply(self, mods):
        """mods: int32 array of shape (B, 4) = {kind, u, v, w}. Returns (status, first_new_id, bad_index)."""
        m = np.ascontiguousarray(mods, dtype=np.int32).reshape(-1, 4)
        fid = C.c_int64(0)
        bad = C.c_int64(-1)
        s = lib().ora_apply(self.h, _p(m, C.c_int32), len(m), C.byref(fid), C.byref(bad))
        return int(s), int(fid.value), int(bad.value)

    def refine(self):
        st = np.zeros(len(STATS), dtype=np.int64)
        s = lib().ora_refine(self.h, _p(st, C.c_int64))
        return int(s), dict(zip(STATS, (int(x) for x in st)))

    def refine_global(self):
        """NEXT-1: every boundary vertex (adj_ext != 0) joins A, then refine."""
        st = np.zeros(len(STATS), dtype=np.int64)
        s = lib().ora_refine_global(self.h, _p(st, C.c_int64))
        return int(s), dict(zip(STATS, (int(x) for x in st)))

    def repartition(self, group_size: int = 6) -> int:
        """NEXT-2 reading F8: full FGP repartition of the current graph in place (status)."""
        return int(lib().ora_repartition(self.h, group_size))

    @property
    def n_total(self):
        return int(lib().ora_n_total(self.h))

    @property
    def n_active(self):
        return int(lib().ora_n_active(self.h))

    def partition(self):
        out = np.empty(self.n_total, dtype=np.int32)
        lib().ora_partition(self.h, _p(out, C.c_int32))
        return out

    def cut(self):
        return int(lib().ora_cut(self.h))

    def part_weights(self):
        out = np.empty(self.k, dtype=np.int64)
        lib().ora_part_weights(self.h, _p(out, C.c_int64))
        return out

    def total_weight(self):
        return int(lib().ora_total_weight(self.h))

    def cap(self):
        return int(lib().ora_cap_value(self.h))

    def export_csr(self):
        n = self.n_total
        m = int(lib().ora_num_slots(self.h))
        xadj = np.empty(n + 1, dtype=np.int64)
        adj = np.empty(max(m, 1), dtype=np.int32)
        w = np.empty(max(m, 1), dtype=np.int32)
        lib().ora_export_csr(self.h, _p(xadj, C.c_int64), _p(adj, C.c_int32), _p(w, C.c_int32))
        return xadj, adj[:m], w[:m]

    def check_invariants(self, reported_cut: int = -1, structure: bool = True):
        """None if I1-I6 hold, else the first violation ("I6: ...", "I5: ...",
        order I6, I5, I2, I3, I4, I1).  I1 compares `reported_cut` (e.g. the
        product's maintained cut) with the oracle's recount; -1 skips it.
        structure=False skips the O(m log m) adjacency check I6."""
        buf = C.create_string_buffer(256)
        r = lib().ora_check_invariants_ext(self.h, int(reported_cut), 0 if structure else 1, buf, 256)
        return None if r == 0 else buf.value.decode()

    # TEST-ONLY corruption hooks: build states violating one invariant
    def debug_set_part(self, v, p):
        lib().ora_debug_set_part(self.h, int(v), int(p))

    def debug_set_part_weight(self, p, w):
        lib().ora_debug_set_part_weight(self.h, int(p), int(w))

    def debug_set_total_weight(self, W):
        lib().ora_debug_set_total_weight(self.h, int(W))

    def debug_set_frontier(self, v, f):
        lib().ora_debug_set_frontier(self.h, int(v), int(bool(f)))

    def debug_add_half_edge(self, u, x, w=1):
        lib().ora_debug_add_half_edge(self.h, int(u), int(x), int(w))

    def debug_set_edge_weight(self, u, x, w):
        lib().ora_debug_set_edge_weight(self.h, int(u), int(x), int(w))

    def trace_rounds(self, maxr=1 << 16):
        S = np.zeros(maxr, dtype=np.int64)
        Lr = np.zeros(maxr, dtype=np.int64)
        r = int(lib().ora_trace_rounds(self.h, _p(S, C.c_int64), _p(Lr, C.c_int64), maxr))
        return S[:r], Lr[:r]

    def trace_moves(self, maxm=1 << 20):
        out = np.zeros(3 * maxm, dtype=np.int64)
        m = int(lib().ora_trace_moves(self.h, _p(out, C.c_int64), 3 * maxm))
        return out[: 3 * m].reshape(m, 3)

    def trace_sets(self):
        n = self.n_total
        a = np.zeros(n, dtype=np.uint8)
        b = np.zeros(n, dtype=np.uint8)
        c = np.zeros(n, dtype=np.uint8)
        lib().ora_trace_sets(self.h, a.ctypes.data, b.ctypes.data, c.ctypes.data)
        return a.astype(bool), b.astype(bool), c.astype(bool)
