"""B200-native iG-kway incremental refinement (libigk.so, sm_100a).

Thin ctypes binding of the C ABI in include/igk.h: argument marshalling only;
every step of apply/refine runs in the CUDA kernels of csrc/.  There is no
CPU fallback: if libigk.so is missing the import fails loudly.
"""
from __future__ import annotations

import ctypes as C
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
# IGK_LIB: load another in-tree build of the same library instead (A/B timing
# of kernel variants by tools/; the product default is libigk.so here)
_SO = os.environ.get("IGK_LIB") or os.path.join(_HERE, "libigk.so")

OK, EINVAL, ENOMEM, ECUDA, ENCCL, ESTATE, WIMBALANCED = 0, 1, 2, 3, 4, 5, 6
EDGE_DELETE, VERTEX_DELETE, VERTEX_INSERT, EDGE_INSERT = 0, 1, 2, 3

STATS = ["affected", "inserted", "expanded", "filtered_in", "expanded_in", "evicted", "rounds",
         "moves_applied", "moves_deferred", "cut", "cap", "max_part_weight", "imbalanced",
         "adj_entries_scanned", "repartitioned"]

# every symbol include/igk.h declares (checked by tests/test_abi.py)
SYMBOLS = ["igk_create", "igk_apply_modifiers", "igk_apply_modifiers_device", "igk_refine", "igk_refine_global",
           "igk_step", "igk_step_device", "igk_nccl_unique_id", "igk_stage_batch", "igk_step_begin",
           "igk_step_end",
           "igk_partition", "igk_partition_delta", "igk_cut_size", "igk_part_weights", "igk_num_vertices", "igk_recount",
           "igk_export_csr", "igk_store_stats", "igk_compact", "igk_kernel_launches", "igk_last_kernel_ms", "igk_debug_phase_times", "igk_debug_arrivals",
           "igk_debug_paths", "igk_debug_set_profile", "igk_debug_phase_work", "igk_fgp_partition", "igk_repartition",
           "igk_last_error", "igk_destroy"]


# igk_debug_paths counters (include/igk.h IGK_PATH_*)
PATHS = ["hub_filter", "hub_commit", "hub_gain", "tie_cta", "tie_grid", "key_exact", "key64", "forced_l0",
         "wfallback", "r3", "r3_key64", "reloc", "vdel_warp", "vdel_thread", "warp_gain", "reserved15",
         "compaction", "vertex_growth", "split_step", "fused_step", "notice_fallback"]


ALLREDUCE_FN = C.CFUNCTYPE(C.c_int32, C.c_void_p, C.c_void_p, C.c_int64, C.c_int32, C.c_int32)


class Comm(C.Structure):
    """igk_comm: host-callback collective of sharded handles (include/igk.h)"""
    _fields_ = [("ctx", C.c_void_p), ("allreduce", ALLREDUCE_FN)]


class Options(C.Structure):
    _fields_ = [("device", C.c_int), ("stream", C.c_void_p), ("max_vertices", C.c_int64),
                ("max_slots", C.c_int64), ("slack_min", C.c_int32), ("validate", C.c_int32),
                ("check_invariants", C.c_int32), ("blocks_per_sm", C.c_int32),
                ("nranks", C.c_int32), ("rank", C.c_int32), ("nccl_id", C.c_void_p),
                ("comm", C.POINTER(Comm)), ("p2p", C.c_int32), ("ranks_per_device", C.c_int32),
                ("wide_weights", C.c_int32), ("fgp_fallback_ppm", C.c_int64)]


class Stats(C.Structure):
    _fields_ = [(s, C.c_int64) for s in STATS]


class TorchComm:
    """igk_comm over torch.distributed (host tensors: the gloo backend), for
    sharded handles without NCCL -- the tests' transport (several ranks on
    one GPU).  Plumbing only: the library hands it host buffers of fixed
    size (candidate bitmaps, restoration keys, move records, scalars) to
    all-reduce; every value is produced and consumed by the CUDA kernels."""

    _DT = {0: ("int64", 8), 1: ("uint32", 4)}

    def __init__(self, group=None):
        import torch.distributed as dist
        self.dist, self.group = dist, group
        self.nranks = dist.get_world_size(group)
        self.rank = dist.get_rank(group)
        self.calls = 0
        self._cb = ALLREDUCE_FN(self._allreduce)
        self.struct = Comm(None, self._cb)

    def _allreduce(self, ctx, buf, count, dtype, op):
        try:
            import torch
            name, size = self._DT[dtype]
            arr = np.ctypeslib.as_array((C.c_uint8 * (count * size)).from_address(buf)).view(name)
            # gloo has no uint32: reduce the bit patterns as int64 (values < 2^32, at most one
            # non-zero contribution per element for SUM, or a MIN / MAX of non-negative values)
            t = torch.from_numpy(arr.astype(np.int64))
            red = {0: self.dist.ReduceOp.SUM, 1: self.dist.ReduceOp.MIN, 2: self.dist.ReduceOp.MAX}[op]
            self.dist.all_reduce(t, op=red, group=self.group)
            arr[:] = t.numpy().astype(name)
            self.calls += 1
            return 0
        except Exception:  # never let an exception cross the C ABI
            import traceback
            traceback.print_exc()
            return -1


class IGKError(RuntimeError):
    def __init__(self, status, msg):
        super().__init__(f"igk status {status}: {msg}")
        self.status = status


_lib = None


def lib():
    """Load libigk.so (fails loudly if it was not built)."""
    global _lib
    if _lib is None:
        if not os.path.exists(_SO):
            raise ImportError(f"{_SO} is missing: build it with `python -m "
                              "paper_conf_dac_leejlczcshh25_b200.build` (no CPU fallback exists)")
        L = C.CDLL(_SO)
        P, i64, i32 = C.c_void_p, C.c_int64, C.c_int32
        i64p, i32p = C.POINTER(C.c_int64), C.POINTER(C.c_int32)
        L.igk_create.restype = C.c_int
        L.igk_create.argtypes = [C.POINTER(Options), i64, i64p, i32p, i32p, i32p, i32, C.c_double, i32p,
                                 C.POINTER(P)]
        L.igk_apply_modifiers.restype = C.c_int
        L.igk_apply_modifiers.argtypes = [P, P, i64, i64p, i64p]
        L.igk_apply_modifiers_device.restype = C.c_int
        L.igk_apply_modifiers_device.argtypes = [P, P, i64, i64p, i64p]
        L.igk_refine.restype = C.c_int
        L.igk_refine.argtypes = [P, C.POINTER(Stats)]
        L.igk_refine_global.restype = C.c_int
        L.igk_refine_global.argtypes = [P, C.POINTER(Stats)]
        L.igk_step.restype = C.c_int
        L.igk_step.argtypes = [P, P, i64, C.POINTER(Stats), i64p, i64p]
        L.igk_step_device.restype = C.c_int
        L.igk_step_device.argtypes = [P, P, i64, C.POINTER(Stats), i64p, i64p]
        L.igk_stage_batch.restype = C.c_int
        L.igk_stage_batch.argtypes = [P, P, i64]
        L.igk_step_begin.restype = C.c_int
        L.igk_step_begin.argtypes = [P]
        L.igk_step_end.restype = C.c_int
        L.igk_step_end.argtypes = [P, C.POINTER(Stats), i64p, i64p]
        L.igk_nccl_unique_id.restype = C.c_int
        L.igk_nccl_unique_id.argtypes = [P, i64]
        L.igk_partition.restype = C.c_int
        L.igk_partition.argtypes = [P, i32p, i64, i64p]
        L.igk_partition_delta.restype = C.c_int
        L.igk_partition_delta.argtypes = [P, P, i64, i64p]
        L.igk_debug_paths.restype = C.c_int32
        L.igk_debug_paths.argtypes = [P, i64p, C.c_int32]
        L.igk_debug_set_profile.restype = C.c_int
        L.igk_debug_set_profile.argtypes = [P, C.c_int32]
        L.igk_debug_phase_work.restype = C.c_int32
        L.igk_debug_phase_work.argtypes = [P, i64p, i64p, C.c_int32]
        L.igk_cut_size.restype = C.c_int
        L.igk_cut_size.argtypes = [P, i64p]
        L.igk_part_weights.restype = C.c_int
        L.igk_part_weights.argtypes = [P, i64p]
        L.igk_num_vertices.restype = C.c_int
        L.igk_num_vertices.argtypes = [P, i64p, i64p]
        L.igk_recount.restype = C.c_int
        L.igk_recount.argtypes = [P, i64p, i64p]
        L.igk_export_csr.restype = C.c_int
        L.igk_export_csr.argtypes = [P, i64p, i64, i32p, i32p, i64, i64p, i64p]
        L.igk_store_stats.restype = C.c_int
        L.igk_store_stats.argtypes = [P, i64p, i64p, i64p, i64p, i64p]
        L.igk_compact.restype = C.c_int
        L.igk_compact.argtypes = [P]
        L.igk_kernel_launches.restype = i64
        L.igk_kernel_launches.argtypes = [P]
        L.igk_last_kernel_ms.restype = C.c_int
        L.igk_last_kernel_ms.argtypes = [P, C.POINTER(C.c_float), C.POINTER(C.c_float), C.POINTER(C.c_float)]
        L.igk_debug_phase_times.restype = C.c_int32
        L.igk_debug_phase_times.argtypes = [P, C.c_int32, i32p, i64p, C.c_int32]
        L.igk_debug_arrivals.restype = C.c_int32
        L.igk_debug_arrivals.argtypes = [P, C.c_int32, i64p, C.c_int32]
        L.igk_fgp_partition.restype = C.c_int
        L.igk_fgp_partition.argtypes = [C.POINTER(Options), i64, i64p, i32p, i32p, i32p, i32, C.c_double, i32,
                                        i32p, i64p, i32p]
        L.igk_repartition.restype = C.c_int
        L.igk_repartition.argtypes = [P, C.c_int32, i64p]
        L.igk_last_error.restype = C.c_char_p
        L.igk_last_error.argtypes = [P]
        L.igk_destroy.restype = None
        L.igk_destroy.argtypes = [P]
        _lib = L
    return _lib


def _p(a, ct):
    return None if a is None else a.ctypes.data_as(C.POINTER(ct))


def nccl_unique_id() -> bytes:
    """ncclUniqueId (128 bytes) for sharded handles: create on one rank, share."""
    buf = C.create_string_buffer(128)
    s = lib().igk_nccl_unique_id(buf, 128)
    if s != OK:
        raise IGKError(s, "igk_nccl_unique_id failed (NCCL not loadable?)")
    return buf.raw


def fgp_partition(xadj, adjncy, k, eps, vwgt=None, adjwgt=None, group_size=6, device=0, stream=None):
    """Full k-way partition on the GPU (igk_fgp_partition, IGK-FGP v1).

    Returns (part int32[n], level sizes list)."""
    xadj = np.ascontiguousarray(xadj, dtype=np.int64)
    adjncy = np.ascontiguousarray(adjncy, dtype=np.int32)
    vwgt = None if vwgt is None else np.ascontiguousarray(vwgt, dtype=np.int32)
    adjwgt = None if adjwgt is None else np.ascontiguousarray(adjwgt, dtype=np.int32)
    n = len(xadj) - 1
    o = Options()
    o.device = device
    o.stream = stream or 0
    part = np.empty(max(n, 1), np.int32)
    lv = np.zeros(40, np.int64)
    nl = C.c_int32(0)
    s = lib().igk_fgp_partition(C.byref(o), n, _p(xadj, C.c_int64), _p(adjncy, C.c_int32), _p(vwgt, C.c_int32),
                                _p(adjwgt, C.c_int32), k, eps, group_size, _p(part, C.c_int32),
                                _p(lv, C.c_int64), C.byref(nl))
    if s != OK:
        raise IGKError(s, (lib().igk_last_error(None) or b"").decode())
    return part[:n], [int(x) for x in lv[:nl.value]]


class IGKGraph:
    """One GPU-resident graph + k-way partition (igk_create)."""

    def __init__(self, xadj, adjncy, k, eps, part, vwgt=None, adjwgt=None, device=0, stream=None,
                 max_vertices=0, max_slots=0, slack_min=0, check=False, blocks_per_sm=0,
                 nranks=1, rank=0, nccl_id: bytes | None = None, comm=None, p2p=False, ranks_per_device=1, wide_weights=False,
                 fgp_fallback: float = 0.0):
        """nranks > 1: rank `rank` of a vertex-range sharded graph (collective
        calls; every rank passes the same graph and batches).  Transport: NCCL
        from `nccl_id` (nccl_unique_id() on one rank, shared), else `comm`.
        fgp_fallback > 0: full repartition once the accepted modifiers reach
        that fraction of |V| (e.g. 0.5)."""
        L = lib()
        xadj = np.ascontiguousarray(xadj, dtype=np.int64)
        adjncy = np.ascontiguousarray(adjncy, dtype=np.int32)
        part = np.ascontiguousarray(part, dtype=np.int32)
        vwgt = None if vwgt is None else np.ascontiguousarray(vwgt, dtype=np.int32)
        adjwgt = None if adjwgt is None else np.ascontiguousarray(adjwgt, dtype=np.int32)
        self._id = None if nccl_id is None else C.create_string_buffer(bytes(nccl_id), 128)
        self._comm = comm  # keeps the callback alive as long as the handle
        o = Options(device, stream or None, max_vertices, max_slots, slack_min, 1, int(check), blocks_per_sm,
                    int(nranks), int(rank), None if self._id is None else C.cast(self._id, C.c_void_p),
                    None if comm is None else C.pointer(comm.struct), int(bool(p2p)), int(ranks_per_device),
                    int(bool(wide_weights)), int(round(fgp_fallback * 1e6)))
        h = C.c_void_p()
        s = L.igk_create(C.byref(o), len(xadj) - 1, _p(xadj, C.c_int64), _p(adjncy, C.c_int32),
                         _p(vwgt, C.c_int32), _p(adjwgt, C.c_int32), k, eps, _p(part, C.c_int32), C.byref(h))
        if s != OK:
            raise IGKError(s, "igk_create failed: " + L.igk_last_error(None).decode())
        self._destroy = L.igk_destroy  # kept: module globals may be gone at interpreter exit
        self.h = h
        self.k = int(k)

    def close(self):
        if getattr(self, "h", None):
            self._destroy(self.h)
            self.h = None

    __del__ = close

    def _err(self):
        return lib().igk_last_error(self.h).decode()

    def apply(self, mods):
        m = np.ascontiguousarray(mods, dtype=np.int32).reshape(-1, 4)
        fid, bad = C.c_int64(0), C.c_int64(-1)
        s = lib().igk_apply_modifiers(self.h, m.ctypes.data, len(m), C.byref(fid), C.byref(bad))
        return s, fid.value, bad.value

    def apply_device(self, ptr: int, count: int):
        """mods already in device memory (e.g. torch int32 (B,4) tensor .data_ptr())."""
        fid, bad = C.c_int64(0), C.c_int64(-1)
        s = lib().igk_apply_modifiers_device(self.h, C.c_void_p(ptr), count, C.byref(fid), C.byref(bad))
        return s, fid.value, bad.value

    def refine(self):
        st = Stats()
        s = lib().igk_refine(self.h, C.byref(st))
        if s not in (OK, WIMBALANCED):
            raise IGKError(s, self._err())
        return s, {f: int(getattr(st, f)) for f in STATS}

    def repartition(self, group_size: int = 6) -> int:
        """igk_repartition: full FGP repartition of the current graph in place; returns the new cut."""
        cut = C.c_int64(0)
        s = lib().igk_repartition(self.h, group_size, C.byref(cut))
        if s != OK:
            raise IGKError(s, self._err())
        return int(cut.value)

    def refine_global(self):
        """igk_refine_global: the partition boundary (adj_ext != 0) joins A, then refine."""
        st = Stats()
        s = lib().igk_refine_global(self.h, C.byref(st))
        if s not in (OK, WIMBALANCED):
            raise IGKError(s, self._err())
        return s, {f: int(getattr(st, f)) for f in STATS}

    def step(self, mods):
        """apply + refine fused (host batch). Returns (status, stats, bad_index)."""
        m = np.ascontiguousarray(mods, dtype=np.int32).reshape(-1, 4)
        st = Stats()
        fid, bad = C.c_int64(0), C.c_int64(-1)
        s = lib().igk_step(self.h, m.ctypes.data, len(m), C.byref(st), C.byref(fid), C.byref(bad))
        if s not in (OK, WIMBALANCED, EINVAL):
            raise IGKError(s, self._err())
        return s, {f: int(getattr(st, f)) for f in STATS}, bad.value

    def step_device(self, ptr: int, count: int, stats: "Stats | None" = None):
        """apply + refine fused, batch already in device memory.  Returns (status, Stats)."""
        st = stats or Stats()
        fid, bad = C.c_int64(0), C.c_int64(-1)
        s = lib().igk_step_device(self.h, C.c_void_p(ptr), count, C.byref(st), C.byref(fid), C.byref(bad))
        if s not in (OK, WIMBALANCED, EINVAL):
            raise IGKError(s, self._err())
        return s, st

    def stage_batch(self, mods):
        """igk_stage_batch: async H2D of the next batch (keep `mods` alive and
        unchanged until the step_end of the step that consumes it)."""
        m = np.ascontiguousarray(mods, dtype=np.int32).reshape(-1, 4)
        self._staged_keep = getattr(self, "_staged_keep", [])[-1:] + [m]
        s = lib().igk_stage_batch(self.h, m.ctypes.data, len(m))
        if s != OK:
            raise IGKError(s, self._err())

    def step_begin(self):
        s = lib().igk_step_begin(self.h)
        if s != OK:
            raise IGKError(s, self._err())

    def step_end(self):
        """-> (status, stats, bad_index) exactly as step()"""
        st = Stats()
        fid, bad = C.c_int64(0), C.c_int64(-1)
        s = lib().igk_step_end(self.h, C.byref(st), C.byref(fid), C.byref(bad))
        if s not in (OK, WIMBALANCED, EINVAL):
            raise IGKError(s, self._err())
        return s, {f: int(getattr(st, f)) for f in STATS}, bad.value

    def num_vertices(self):
        nt, na = C.c_int64(0), C.c_int64(0)
        s = lib().igk_num_vertices(self.h, C.byref(nt), C.byref(na))
        if s != OK:
            raise IGKError(s, self._err())
        return nt.value, na.value

    def partition(self):
        nt = C.c_int64(0)
        lib().igk_partition(self.h, None, 0, C.byref(nt))
        out = np.empty(max(nt.value, 1), dtype=np.int32)
        s = lib().igk_partition(self.h, _p(out, C.c_int32), len(out), C.byref(nt))
        if s != OK:
            raise IGKError(s, self._err())
        return out[: nt.value]

    def partition_delta(self, out: "np.ndarray | None" = None):
        """(count, 2) int32 array of (vertex, new part) of the last refine / step
        (igk_partition_delta).  `out`: optional (cap, 2) int32 buffer to fill
        (page-locked memory is DMA'd directly); returns a view of it."""
        cnt = C.c_int64(0)
        L = lib()
        if out is None:
            L.igk_partition_delta(self.h, None, 0, C.byref(cnt))
            out = np.empty((max(cnt.value, 1), 2), dtype=np.int32)
        s = L.igk_partition_delta(self.h, C.c_void_p(out.ctypes.data), len(out), C.byref(cnt))
        if s != OK:
            raise IGKError(s, self._err())
        return out[: cnt.value]

    PHASES = ["boundary", "F0_filter", "F1_commit_expand", "F2_filter", "F3_commit", "R3_restore",
              "round_gain", "round_move"]

    def set_profile(self, on: bool = True):
        """profile mode: phase stamps + per-phase work counters on every refine"""
        s = lib().igk_debug_set_profile(self.h, int(bool(on)))
        if s != OK:
            raise IGKError(s, self._err())

    def phase_work(self):
        """{phase: (adjacency entries scanned, list items)} of the last refine (profile mode)"""
        sc = np.zeros(8, np.int64)
        it = np.zeros(8, np.int64)
        n = lib().igk_debug_phase_work(self.h, _p(sc, C.c_int64), _p(it, C.c_int64), 8)
        return {self.PHASES[i]: (int(sc[i]), int(it[i])) for i in range(n)}

    def debug_paths(self):
        """{path name: count} of the device / host path counters (igk_debug_paths)."""
        out = np.zeros(32, np.int64)
        n = lib().igk_debug_paths(self.h, _p(out, C.c_int64), 32)
        return {PATHS[i]: int(out[i]) for i in range(min(n, len(PATHS)))}

    def cut(self):
        c = C.c_int64(0)
        s = lib().igk_cut_size(self.h, C.byref(c))
        if s != OK:
            raise IGKError(s, self._err())
        return c.value

    def part_weights(self):
        out = np.zeros(self.k, dtype=np.int64)
        s = lib().igk_part_weights(self.h, _p(out, C.c_int64))
        if s != OK:
            raise IGKError(s, self._err())
        return out

    def recount(self):
        c = C.c_int64(0)
        wp = np.zeros(self.k, dtype=np.int64)
        s = lib().igk_recount(self.h, C.byref(c), _p(wp, C.c_int64))
        if s != OK:
            raise IGKError(s, self._err())
        return c.value, wp

    def export_csr(self, sort_rows=True):
        nt, ns = C.c_int64(0), C.c_int64(0)
        L = lib()
        L.igk_export_csr(self.h, None, 0, None, None, 0, C.byref(nt), C.byref(ns))
        xadj = np.empty(nt.value + 1, dtype=np.int64)
        adj = np.empty(max(ns.value, 1), dtype=np.int32)
        w = np.empty(max(ns.value, 1), dtype=np.int32)
        s = L.igk_export_csr(self.h, _p(xadj, C.c_int64), len(xadj), _p(adj, C.c_int32), _p(w, C.c_int32),
                             len(adj), C.byref(nt), C.byref(ns))
        if s != OK:
            raise IGKError(s, self._err())
        adj, w = adj[: ns.value], w[: ns.value]
        if sort_rows:
            for u in range(nt.value):
                a, b = xadj[u], xadj[u + 1]
                if b - a > 1:
                    o = np.argsort(adj[a:b], kind="stable")
                    adj[a:b] = adj[a:b][o]
                    w[a:b] = w[a:b][o]
        return xadj, adj, w

    def store_stats(self):
        v = [C.c_int64(0) for _ in range(5)]
        s = lib().igk_store_stats(self.h, *[C.byref(x) for x in v])
        if s != OK:
            raise IGKError(s, self._err())
        return dict(zip(["n_total", "n_active", "adj_entries", "slab_top", "slab_cap"], [x.value for x in v]))

    def compact(self):
        s = lib().igk_compact(self.h)
        if s != OK:
            raise IGKError(s, self._err())

    def kernel_launches(self):
        return int(lib().igk_kernel_launches(self.h))

    def phase_times(self, which):
        """[(phase id, ns since kernel start)] of the last apply (0) / refine (1) kernel."""
        ids = np.zeros(128, np.int32)
        ts = np.zeros(128, np.int64)
        n = lib().igk_debug_phase_times(self.h, which, _p(ids, C.c_int32), _p(ts, C.c_int64), 128)
        return list(zip(ids[:n].tolist(), ts[:n].tolist()))

    def arrivals(self, which):
        """(128, grid) per-CTA barrier arrival stamps (needs IGK_DEBUG_ARRIVALS at create);
        which = 2: (2, warps) per-warp end times / heaviest prefix of the last F1 commit pass."""
        out = np.zeros(128 * 4096, np.int64)
        gsz = lib().igk_debug_arrivals(self.h, which, _p(out, C.c_int64), len(out))
        if which == 2:
            return np.stack([out[j * 4096:j * 4096 + gsz] for j in range(4)]) if gsz else None
        return out[: 128 * gsz].reshape(128, gsz) if gsz else None

    def last_ms(self):
        r, a, c = C.c_float(0), C.c_float(0), C.c_float(0)
        lib().igk_last_kernel_ms(self.h, C.byref(r), C.byref(a), C.byref(c))
        return {"refine": r.value, "apply": a.value, "recount": c.value}
