"""Thin Python binding of the C ABI in include/gp.h (argument marshalling only).

Every step of the coarsening path runs in libgpcoarsen.so's sm_100a kernels; this module
only passes pointers (torch tensors' ``data_ptr()``), sizes and the current CUDA stream.
There is NO CPU fallback: importing this module raises if the shared library is missing,
and creating a context raises if no CUDA device is present.

Names follow the ABI (and the paper's notation: adjp/adjncy/adjwgt/vwgt, P16.s17-19;
match M and cmap CM, P16.s24).
"""
from __future__ import annotations

import ctypes
import os
import weakref
from dataclasses import dataclass
from typing import Dict, List, Optional

import torch

from ._build import LIB

if not os.path.exists(LIB):
    raise ImportError(f"libgpcoarsen.so not built ({LIB}); run __graft_entry__.build() — "
                      "there is no CPU fallback for the coarsening path")

_lib = ctypes.CDLL(LIB)

_vp = ctypes.c_void_p
_i32 = ctypes.c_int32
_i32p = ctypes.POINTER(ctypes.c_int32)

GP_INPUT_DEVICE = 0x1
GP_VALIDATE = 0x2

STATUS = {0: "GP_OK", 1: "GP_ERR_INVALID_ARG", 2: "GP_ERR_INVALID_GRAPH", 3: "GP_ERR_OVERFLOW",
          4: "GP_ERR_OUT_OF_MEMORY", 5: "GP_ERR_CUDA", 6: "GP_ERR_NCCL", 7: "GP_ERR_INTERNAL"}

STOP_NONE, STOP_THRESHOLD, STOP_STALL, STOP_MAX_LEVELS = 0, 1, 2, 3
K_PROPOSE, K_COMMIT, K_CMAP, K_CONTRACT, K_ASSEMBLE, K_OTHER = range(6)
KERNEL_KINDS = ["propose", "commit", "cmap", "contract", "assemble", "other"]


class GPError(RuntimeError):
    def __init__(self, status: int, where: str):
        detail = _lib.gp_last_error().decode(errors="replace")
        super().__init__(f"{where}: {STATUS.get(status, status)}: {detail}")
        self.status = status


class CoarsenOpts(ctypes.Structure):
    _fields_ = [("threshold", _i32), ("stall_ratio_pct", _i32), ("max_levels", _i32), ("max_rounds", _i32),
                ("tie_seed", ctypes.c_uint32)]


class Level(ctypes.Structure):
    _fields_ = [("n", _i32), ("nnz", _i32), ("n_coarse", _i32), ("cnnz", _i32), ("rounds", _i32),
                ("maximal", _i32), ("stop_reason", _i32), ("reserved", _i32),
                ("arcs_scanned", ctypes.c_int64), ("rows_scanned", ctypes.c_int64),
                ("live_visits", ctypes.c_int64), ("d_match", _vp), ("d_cmap", _vp), ("coarse", _vp),
                ("v_begin", _i32), ("n_local", _i32), ("cv_begin", _i32), ("n_coarse_local", _i32)]


class RefineOpts(ctypes.Structure):
    _fields_ = [("nparts", _i32), ("imbalance_pct", _i32), ("max_passes", _i32)]


class KernelStats(ctypes.Structure):
    _fields_ = [("launches", ctypes.c_int64), ("ms", ctypes.c_double)]


def _sig(name, res, args):
    f = getattr(_lib, name)
    f.restype = res
    f.argtypes = args
    return f


_sig("gp_status_string", ctypes.c_char_p, [ctypes.c_int])
_sig("gp_last_error", ctypes.c_char_p, [])
_sig("gp_ctx_create", ctypes.c_int, [ctypes.c_int, _vp, ctypes.POINTER(_vp)])
# gp_alloc_fn / gp_dealloc_fn (include/gp.h)
ALLOC_FN = ctypes.CFUNCTYPE(_vp, ctypes.c_size_t, _vp, _vp)
DEALLOC_FN = ctypes.CFUNCTYPE(None, _vp, _vp, _vp)
_sig("gp_ctx_set_allocator", ctypes.c_int, [_vp, ALLOC_FN, DEALLOC_FN, _vp])
_sig("gp_ctx_num_sms", ctypes.c_int, [_vp, _i32p])
_sig("gp_graph_create", ctypes.c_int, [_vp, _i32, _vp, _vp, _vp, _vp, ctypes.c_uint32, ctypes.POINTER(_vp)])
_sig("gp_graph_view", ctypes.c_int, [_vp, _i32p, _i32p, ctypes.POINTER(_vp), ctypes.POINTER(_vp),
                                     ctypes.POINTER(_vp), ctypes.POINTER(_vp)])
_sig("gp_graph_download", ctypes.c_int, [_vp, _vp, _vp, _vp, _vp])
_sig("gp_match_level", ctypes.c_int, [_vp, _vp, _i32, _i32p])
_sig("gp_match_level_ex", ctypes.c_int, [_vp, _vp, _i32, ctypes.c_uint32, _i32p])
_sig("gp_contract_level", ctypes.c_int, [_vp, _vp, _vp, ctypes.POINTER(_vp)])
_sig("gp_coarsen_to", ctypes.c_int, [_vp, ctypes.POINTER(CoarsenOpts), ctypes.POINTER(_vp)])
_sig("gp_hier_num_levels", ctypes.c_int, [_vp, _i32p])
_sig("gp_hier_level", ctypes.c_int, [_vp, _i32, ctypes.POINTER(Level)])
_sig("gp_hier_download_level", ctypes.c_int, [_vp, _i32, _vp, _vp])
_sig("gp_hier_download_coarse", ctypes.c_int, [_vp, _i32, _vp, _vp, _vp, _vp, _i32p, _i32p])
_sig("gp_nccl_unique_id", ctypes.c_int, [_vp])
_sig("gp_project", ctypes.c_int, [_vp, _i32, _i32, _vp, _vp])
_sig("gp_refine", ctypes.c_int, [_vp, _vp, ctypes.POINTER(RefineOpts), _i32p, _i32p])
_sig("gp_uncoarsen", ctypes.c_int, [_vp, _vp, _vp, _vp, ctypes.POINTER(RefineOpts), _i32p])
_sig("gp_ctx_create_dist", ctypes.c_int, [ctypes.c_int, _vp, _vp, ctypes.c_int, ctypes.c_int, ctypes.POINTER(_vp)])
_sig("gp_ctx_create_loopback", ctypes.c_int, [ctypes.c_int, _vp, ctypes.c_int, ctypes.POINTER(_vp)])
_sig("gp_ctx_dist_info", ctypes.c_int, [_vp, _i32p, _i32p])
_sig("gp_graph_create_dist", ctypes.c_int, [_vp, _i32, _i32, _i32, _vp, _vp, _vp, _vp, ctypes.c_uint32,
                                            ctypes.POINTER(_vp)])
_sig("gp_free", None, [_vp])
_sig("gp_ctx_set_timing", ctypes.c_int, [_vp, _i32])
_sig("gp_ctx_kernel_stats", ctypes.c_int, [_vp, ctypes.c_int, ctypes.POINTER(KernelStats)])
_sig("gp_ctx_reset_stats", ctypes.c_int, [_vp])
_sig("gp_ctx_launch_count", ctypes.c_int, [_vp, ctypes.POINTER(ctypes.c_int64)])
_sig("gp_ctx_launch_times", ctypes.c_int, [_vp, _i32, _vp, _vp, _i32p])


def _check(st: int, where: str) -> None:
    if st != 0:
        raise GPError(st, where)


def _ptr(t: Optional[torch.Tensor]):
    if t is None:
        return None
    assert t.dtype == torch.int32 and t.is_contiguous(), "int32 contiguous tensors expected"
    return t.data_ptr()


def nccl_unique_id() -> bytes:
    """gp_nccl_unique_id: the 128-byte NCCL id rank 0 creates and broadcasts."""
    buf = ctypes.create_string_buffer(128)
    _check(_lib.gp_nccl_unique_id(buf), "gp_nccl_unique_id")
    return buf.raw


class Context:
    """gp_ctx on a CUDA device, enqueuing on the given (default: current) torch stream.

    Context(dev)                           single GPU
    Context(dev, loopback=G)               G simulated ranks of the sharded path on one GPU
    Context(dev, nccl_id=id, rank=r, nranks=G)   rank r of G processes (one per GPU, NCCL)
    """

    def __init__(self, device: int = 0, stream: Optional[torch.cuda.Stream] = None, *, loopback: int = 0,
                 nccl_id: Optional[bytes] = None, rank: int = 0, nranks: int = 1):
        if not torch.cuda.is_available():
            raise RuntimeError("no CUDA device: the coarsening path has no CPU fallback")
        self.device = device
        self.stream = stream if stream is not None else torch.cuda.current_stream(device)
        h = _vp()
        if nccl_id is not None:
            idbuf = ctypes.create_string_buffer(bytes(nccl_id), 128)
            _check(_lib.gp_ctx_create_dist(device, self.stream.cuda_stream, idbuf, rank, nranks, ctypes.byref(h)),
                   "gp_ctx_create_dist")
        elif loopback:
            _check(_lib.gp_ctx_create_loopback(device, self.stream.cuda_stream, loopback, ctypes.byref(h)),
                   "gp_ctx_create_loopback")
        else:
            _check(_lib.gp_ctx_create(device, self.stream.cuda_stream, ctypes.byref(h)), "gp_ctx_create")
        self.handle = h
        self._children = weakref.WeakSet()  # live Graph / Hierarchy objects (closed before the context)
        self._alloc_cbs = None              # keeps the ctypes allocator callbacks alive

    def _h(self):
        if self.handle is None or not self.handle.value:
            raise RuntimeError("gp context is closed")
        return self.handle

    def _adopt(self, obj) -> None:
        self._children.add(obj)

    def set_allocator(self, alloc=None, dealloc=None) -> None:
        """gp_ctx_set_allocator: route the library's device allocations through Python
        callables alloc(nbytes, stream) -> int pointer and dealloc(ptr, stream); None restores
        cudaMallocAsync.  Refused (GPError) while graphs or hierarchies of this context are alive."""
        if (alloc is None) != (dealloc is None):
            raise ValueError("alloc and dealloc go together")
        if alloc is None:
            cbs = (ctypes.cast(None, ALLOC_FN), ctypes.cast(None, DEALLOC_FN))
        else:
            def _a(nbytes, stream, user):
                try:
                    return int(alloc(int(nbytes), stream))
                except Exception:  # the library reports GP_ERR_OUT_OF_MEMORY
                    return None

            def _d(ptr, stream, user):
                try:
                    dealloc(ptr, stream)
                except Exception:
                    pass
            cbs = (ALLOC_FN(_a), DEALLOC_FN(_d))
        _check(_lib.gp_ctx_set_allocator(self._h(), cbs[0], cbs[1], None), "gp_ctx_set_allocator")
        self._alloc_cbs = cbs

    def use_torch_allocator(self) -> None:
        """Allocate through torch's caching allocator (stream-ordered on the context stream)."""
        dev = self.device
        self.set_allocator(lambda n, stream: torch.cuda.caching_allocator_alloc(n, dev, stream),
                           lambda p, stream: torch.cuda.caching_allocator_delete(p))

    def dist_info(self):
        """(rank, nranks): (0, 1) single GPU, (-1, G) loopback."""
        r, g = _i32(), _i32()
        _check(_lib.gp_ctx_dist_info(self.handle, ctypes.byref(r), ctypes.byref(g)), "gp_ctx_dist_info")
        return r.value, g.value

    def close(self) -> None:
        """Free the context; its live hierarchies and graphs are closed first (gp.h: a graph
        or hierarchy must be freed before its context)."""
        if self.handle is not None and self.handle.value:
            kids = list(getattr(self, "_children", ()))
            for k in kids:
                if isinstance(k, Hierarchy):
                    k.close()
            for k in kids:
                k.close()
            _lib.gp_free(self.handle)
        self.handle = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    @property
    def num_sms(self) -> int:
        v = _i32()
        _check(_lib.gp_ctx_num_sms(self.handle, ctypes.byref(v)), "gp_ctx_num_sms")
        return v.value

    def set_timing(self, on: bool) -> None:
        _check(_lib.gp_ctx_set_timing(self.handle, 1 if on else 0), "gp_ctx_set_timing")

    def reset_stats(self) -> None:
        _check(_lib.gp_ctx_reset_stats(self.handle), "gp_ctx_reset_stats")

    def kernel_stats(self) -> Dict[str, Dict[str, float]]:
        out = {}
        for k, name in enumerate(KERNEL_KINDS):
            s = KernelStats()
            _check(_lib.gp_ctx_kernel_stats(self.handle, k, ctypes.byref(s)), "gp_ctx_kernel_stats")
            out[name] = {"launches": int(s.launches), "ms": float(s.ms)}
        return out

    def launch_times(self):
        """[(kind name, ms)] of every timed launch since the last reset_stats (launch order)."""
        cnt = _i32()
        _check(_lib.gp_ctx_launch_times(self.handle, 0, None, None, ctypes.byref(cnt)), "gp_ctx_launch_times")
        n = cnt.value
        kinds = (ctypes.c_int32 * max(n, 1))()
        ms = (ctypes.c_float * max(n, 1))()
        _check(_lib.gp_ctx_launch_times(self.handle, n, kinds, ms, ctypes.byref(cnt)), "gp_ctx_launch_times")
        return [(KERNEL_KINDS[kinds[i]], float(ms[i])) for i in range(min(n, cnt.value))]

    def launch_count(self) -> int:
        v = ctypes.c_int64()
        _check(_lib.gp_ctx_launch_count(self.handle, ctypes.byref(v)), "gp_ctx_launch_count")
        return int(v.value)


class Graph:
    """Library-owned device CSR graph (gp_graph)."""

    def __init__(self, ctx: Context, handle, owned: bool = True, parent: Optional["Hierarchy"] = None):
        self.ctx = ctx
        self.handle = handle
        self.owned = owned
        self.parent = parent  # a borrowed level graph keeps its hierarchy alive
        if owned:
            ctx._adopt(self)

    def _h(self):
        if self.handle is None or not self.handle.value:
            raise RuntimeError("gp graph is closed")
        if self.parent is not None and self.parent.handle is None:
            raise RuntimeError("gp graph belongs to a hierarchy that was closed")
        if self.ctx.handle is None:
            raise RuntimeError("gp context is closed")
        return self.handle

    @classmethod
    def create(cls, ctx: Context, adjp: torch.Tensor, adjncy: torch.Tensor, adjwgt: Optional[torch.Tensor] = None,
               vwgt: Optional[torch.Tensor] = None, validate: bool = False) -> "Graph":
        """gp_graph_create from int32 tensors, all on the GPU or all on the host (pinned
        host memory gives asynchronous copies)."""
        n = adjp.numel() - 1
        dev = adjp.is_cuda
        for t in (adjncy, adjwgt, vwgt):
            if t is not None and t.is_cuda != dev:
                raise ValueError("inputs must all be on the device or all on the host")
        flags = (GP_INPUT_DEVICE if dev else 0) | (GP_VALIDATE if validate else 0)
        h = _vp()
        _check(_lib.gp_graph_create(ctx._h(), n, _ptr(adjp), _ptr(adjncy), _ptr(adjwgt), _ptr(vwgt), flags,
                                    ctypes.byref(h)), "gp_graph_create")
        return cls(ctx, h)

    @classmethod
    def create_dist(cls, ctx: Context, n_global: int, v_begin: int, adjp_local: torch.Tensor,
                    adjncy: torch.Tensor, adjwgt: Optional[torch.Tensor] = None,
                    vwgt: Optional[torch.Tensor] = None) -> "Graph":
        """gp_graph_create_dist: this rank's rows [v_begin, v_begin + len(adjp_local) - 1)
        with local offsets and global column ids (collective over the NCCL context)."""
        v_end = v_begin + adjp_local.numel() - 1
        flags = GP_INPUT_DEVICE if adjp_local.is_cuda else 0
        h = _vp()
        _check(_lib.gp_graph_create_dist(ctx._h(), n_global, v_begin, v_end, _ptr(adjp_local), _ptr(adjncy),
                                         _ptr(adjwgt), _ptr(vwgt), flags, ctypes.byref(h)), "gp_graph_create_dist")
        return cls(ctx, h)

    def close(self) -> None:
        if self.owned and self.handle is not None and self.handle.value and self.ctx.handle is not None:
            _lib.gp_free(self.handle)
        self.handle = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def view(self):
        n, nnz = _i32(), _i32()
        _check(_lib.gp_graph_view(self._h(), ctypes.byref(n), ctypes.byref(nnz), None, None, None, None),
               "gp_graph_view")
        return n.value, nnz.value

    @property
    def n(self) -> int:
        return self.view()[0]

    @property
    def nnz(self) -> int:
        return self.view()[1]

    def download(self, out: Optional[Dict[str, torch.Tensor]] = None) -> Dict[str, torch.Tensor]:
        """Copy the CSR arrays to host int32 tensors (gp_graph_download); `out` may supply
        preallocated (e.g. pinned) host tensors of at least the right sizes."""
        n, nnz = self.view()
        if out is None:
            out = {k: torch.empty(sz, dtype=torch.int32) for k, sz in
                   (("adjp", n + 1), ("adjncy", nnz), ("adjwgt", nnz), ("vwgt", n))}
        _check(_lib.gp_graph_download(self._h(), out["adjp"].data_ptr(), out["adjncy"].data_ptr(),
                                      out["adjwgt"].data_ptr(), out["vwgt"].data_ptr()), "gp_graph_download")
        out["n"], out["nnz"] = n, nnz
        return out

    def match_level(self, match: torch.Tensor, max_rounds: int = 0, sync_rounds: bool = True,
                    tie_seed: int = 0) -> Optional[int]:
        """gp_match_level_ex into a caller-owned device int32[n] tensor; returns rounds.
        tie_seed != 0: equal-weight ties go to the lower lowbias32(v ^ seed) (RM, P18.s8)."""
        r = _i32()
        _check(_lib.gp_match_level_ex(self._h(), _ptr(match), max_rounds, tie_seed & 0xFFFFFFFF,
                                      ctypes.byref(r) if sync_rounds else None), "gp_match_level_ex")
        return r.value if sync_rounds else None

    def contract_level(self, match: torch.Tensor, cmap: torch.Tensor) -> "Graph":
        """gp_contract_level: fills cmap, returns the coarse graph (caller-owned)."""
        h = _vp()
        _check(_lib.gp_contract_level(self._h(), _ptr(match), _ptr(cmap), ctypes.byref(h)), "gp_contract_level")
        return Graph(self.ctx, h)

    def refine(self, part: torch.Tensor, nparts: int, imbalance_pct: int = 3, max_passes: int = 8):
        """gp_refine: refine the device int32[n] labelling `part` in place (P22.s1-22);
        returns (moves, passes)."""
        o = RefineOpts(nparts, imbalance_pct, max_passes)
        mv, ps = _i32(), _i32()
        _check(_lib.gp_refine(self._h(), _ptr(part), ctypes.byref(o), ctypes.byref(mv), ctypes.byref(ps)), "gp_refine")
        return mv.value, ps.value

    def coarsen_to(self, threshold: int, stall_ratio_pct: int = 95, max_levels: int = 64,
                   max_rounds: int = 0, tie_seed: int = 0) -> "Hierarchy":
        opts = CoarsenOpts(threshold, stall_ratio_pct, max_levels, max_rounds, tie_seed & 0xFFFFFFFF)
        h = _vp()
        _check(_lib.gp_coarsen_to(self._h(), ctypes.byref(opts), ctypes.byref(h)), "gp_coarsen_to")
        return Hierarchy(self.ctx, h)


@dataclass
class LevelInfo:
    n: int
    nnz: int
    n_coarse: int
    cnnz: int
    rounds: int
    maximal: bool
    stop_reason: int
    arcs_scanned: int
    rows_scanned: int
    live_visits: int
    coarse: Graph
    v_begin: int = 0
    n_local: int = 0
    cv_begin: int = 0
    n_coarse_local: int = 0


class Hierarchy:
    """gp_hier: the kept level hierarchy (M, CM, coarse graph per level; P20.s27)."""

    def __init__(self, ctx: Context, handle):
        self.ctx = ctx
        self.handle = handle
        ctx._adopt(self)

    def _h(self):
        if self.handle is None or not self.handle.value:
            raise RuntimeError("gp hierarchy is closed")
        if self.ctx.handle is None:
            raise RuntimeError("gp context is closed")
        return self.handle

    def close(self) -> None:
        """Free the hierarchy; the borrowed level graphs (LevelInfo.coarse) become unusable."""
        if self.handle is not None and self.handle.value and self.ctx.handle is not None:
            _lib.gp_free(self.handle)
        self.handle = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def __len__(self) -> int:
        v = _i32()
        _check(_lib.gp_hier_num_levels(self._h(), ctypes.byref(v)), "gp_hier_num_levels")
        return v.value

    def level(self, i: int) -> LevelInfo:
        l = Level()
        _check(_lib.gp_hier_level(self._h(), i, ctypes.byref(l)), "gp_hier_level")
        return LevelInfo(l.n, l.nnz, l.n_coarse, l.cnnz, l.rounds, bool(l.maximal), l.stop_reason,
                         l.arcs_scanned, l.rows_scanned, l.live_visits,
                         Graph(self.ctx, _vp(l.coarse), owned=False, parent=self),
                         l.v_begin, l.n_local, l.cv_begin, l.n_coarse_local)

    def levels(self) -> List[LevelInfo]:
        return [self.level(i) for i in range(len(self))]

    def download_level(self, i: int, match: Optional[torch.Tensor] = None, cmap: Optional[torch.Tensor] = None,
                       want_match: bool = True):
        """(match, cmap) of level i as host int32 tensors (optionally preallocated/pinned);
        want_match=False skips the match copy and returns (None, cmap)."""
        info = self.level(i)
        rank, _ = self.ctx.dist_info()
        n = info.n_local if rank >= 0 else info.n  # NCCL rank: its piece; loopback / 1 GPU: all
        m = None if not want_match else (match if match is not None else torch.empty(n, dtype=torch.int32))
        c = cmap if cmap is not None else torch.empty(n, dtype=torch.int32)
        _check(_lib.gp_hier_download_level(self._h(), i, m.data_ptr() if m is not None else None, c.data_ptr()),
               "gp_hier_download_level")
        return m, c


    def project(self, part_coarse: torch.Tensor, part_fine: torch.Tensor, from_level: Optional[int] = None,
                to_level: int = 0) -> torch.Tensor:
        """gp_project: labels of level from_level's coarse graph (default: the coarsest)
        carried down to level to_level's fine graph, written into part_fine (device)."""
        if from_level is None:
            from_level = len(self) - 1
        _check(_lib.gp_project(self._h(), from_level, to_level, _ptr(part_coarse), _ptr(part_fine)), "gp_project")
        return part_fine

    def uncoarsen(self, g0: "Graph", part_coarse: torch.Tensor, part_fine: torch.Tensor, nparts: int,
                  imbalance_pct: int = 3, max_passes: int = 8) -> int:
        """gp_uncoarsen: project + refine level by level from the coarsest labels to level 0
        (written into part_fine); returns the total moves."""
        o = RefineOpts(nparts, imbalance_pct, max_passes)
        mv = _i32()
        _check(_lib.gp_uncoarsen(self._h(), g0._h(), _ptr(part_coarse), _ptr(part_fine), ctypes.byref(o),
                                 ctypes.byref(mv)), "gp_uncoarsen")
        return mv.value

    def download_coarse(self, i: int) -> Dict[str, torch.Tensor]:
        """Coarse graph of level i as host int32 tensors (gp_hier_download_coarse): the whole
        graph on one GPU / loopback, this rank's piece (global column ids) on an NCCL rank."""
        info = self.level(i)
        rank, _ = self.ctx.dist_info()
        n = info.n_coarse_local if rank >= 0 else info.n_coarse
        out = {"adjp": torch.empty(n + 1, dtype=torch.int32), "adjncy": torch.empty(max(info.cnnz, 1), dtype=torch.int32),
               "adjwgt": torch.empty(max(info.cnnz, 1), dtype=torch.int32), "vwgt": torch.empty(max(n, 1), dtype=torch.int32)}
        rows, arcs = _i32(), _i32()
        _check(_lib.gp_hier_download_coarse(self._h(), i, out["adjp"].data_ptr(), out["adjncy"].data_ptr(),
                                            out["adjwgt"].data_ptr(), out["vwgt"].data_ptr(), ctypes.byref(rows),
                                            ctypes.byref(arcs)), "gp_hier_download_coarse")
        out["adjncy"] = out["adjncy"][:arcs.value]
        out["adjwgt"] = out["adjwgt"][:arcs.value]
        out["vwgt"] = out["vwgt"][:rows.value]
        out["n"], out["nnz"] = rows.value, arcs.value
        return out


def exported_symbols():
    """Every gp_* entry point declared in include/gp.h."""
    import re
    hdr = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "include", "gp.h")
    with open(hdr) as f:
        text = f.read()
    text = re.sub(r"/\*.*?\*/", "", text, flags=re.S)               # drop comments
    return sorted(set(re.findall(r"^\s*(?:gp_status|void|const char\s*\*)\s*(gp_[a-z_0-9]+)\s*\(", text,
                                 flags=re.M)))
