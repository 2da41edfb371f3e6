"""Oracle — TEST INFRASTRUCTURE ONLY.

A plain, single-threaded C reference (``oracle/oracle.c``) of the GP-metis coarsening
phase, plus a ctypes binding and the level loop.  Only ``tests/``,
``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` / ``--impl reference``
legs may import this package.  The product path (``paper_conf_ipps_goodarzibg16_b200``)
never imports it and shares no code with it.

Citations are PAPER.md "P<line>.s<k>" sentences; readings R1..R16 are in
DESIGN.md §2.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from typing import Dict, List, Optional

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")
_lib = None

_i32p = ctypes.POINTER(ctypes.c_int32)


def build(force: bool = False) -> str:
    """Compile oracle.c into oracle/liboracle.so with gcc (plain C99, -O2)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-std=c99", "-O2", "-march=native", "-fPIC", "-shared",
                               "-o", tmp, _SRC])
        os.replace(tmp, _LIB)
    return _LIB


def _load():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_LIB)
        lib.oracle_match_level.restype = ctypes.c_int
        lib.oracle_match_level.argtypes = [ctypes.c_int32, _i32p, _i32p, _i32p, ctypes.c_int32,
                                           _i32p, _i32p, _i32p]
        lib.oracle_match_level_seeded.restype = ctypes.c_int
        lib.oracle_match_level_seeded.argtypes = [ctypes.c_int32, _i32p, _i32p, _i32p, ctypes.c_int32,
                                                  ctypes.c_uint32, _i32p, _i32p, _i32p]
        lib.oracle_tie_hash.restype = ctypes.c_uint32
        lib.oracle_tie_hash.argtypes = [ctypes.c_uint32, ctypes.c_uint32]
        lib.oracle_cmap.restype = ctypes.c_int32
        lib.oracle_cmap.argtypes = [ctypes.c_int32, _i32p, _i32p]
        lib.oracle_refine.restype = ctypes.c_int
        lib.oracle_refine.argtypes = [ctypes.c_int32, _i32p, _i32p, _i32p, _i32p, ctypes.c_int32, ctypes.c_int32,
                                      ctypes.c_int32, _i32p, _i32p, _i32p]
        lib.oracle_contract.restype = ctypes.c_int64
        lib.oracle_contract.argtypes = [ctypes.c_int32, _i32p, _i32p, _i32p, _i32p, _i32p, _i32p,
                                        ctypes.c_int32, _i32p, _i32p, _i32p, _i32p]
        _lib = lib
    return _lib


def _np32(a) -> np.ndarray:
    if hasattr(a, "numpy"):
        a = a.detach().cpu().numpy()
    return np.ascontiguousarray(np.asarray(a, dtype=np.int32))


def _p(a: np.ndarray):
    return a.ctypes.data_as(_i32p)


def as_numpy_graph(g: Dict) -> Dict[str, np.ndarray]:
    """CSR dict (torch or numpy arrays) -> int32 numpy arrays."""
    out = {k: _np32(g[k]) for k in ("adjp", "adjncy", "adjwgt", "vwgt")}
    out["n"] = int(len(out["adjp"]) - 1)
    out["nnz"] = int(out["adjp"][-1]) if out["n"] >= 0 and len(out["adjp"]) else 0
    return out


def tie_hash(v: int, seed: int) -> int:
    """RM tie priority h_s(v) of oracle.c (reading R17, P18.s8)."""
    return int(_load().oracle_tie_hash(v & 0xFFFFFFFF, seed & 0xFFFFFFFF))


def match_level(g: Dict, max_rounds: int = 0, tie_seed: int = 0):
    """Heavy-edge handshake matching of one level (oracle.c: oracle_match_level_seeded).
    tie_seed = 0: equal weights go to the lower id (north_star); else to the lower
    h_s(v) (RM reading R17 of P18.s8).

    Returns (match int32[n], rounds, maximal)."""
    lib = _load()
    g = as_numpy_graph(g)
    n = g["n"]
    match = np.empty(max(n, 1), dtype=np.int32)
    rounds = ctypes.c_int32(0)
    maximal = ctypes.c_int32(0)
    st = lib.oracle_match_level_seeded(n, _p(g["adjp"]), _p(g["adjncy"]), _p(g["adjwgt"]),
                                       int(max_rounds), int(tie_seed) & 0xFFFFFFFF, _p(match),
                                       ctypes.byref(rounds), ctypes.byref(maximal))
    if st != 0:
        raise RuntimeError("oracle_match_level: a round with proposals made no match")
    return match[:n], int(rounds.value), bool(maximal.value)


def cmap(match: np.ndarray):
    """Mapping array CM and n_c (oracle.c: oracle_cmap, P18.s16-27)."""
    lib = _load()
    match = _np32(match)
    n = len(match)
    cm = np.empty(max(n, 1), dtype=np.int32)
    n_c = lib.oracle_cmap(n, _p(match), _p(cm))
    return cm[:n], int(n_c)


def contract(g: Dict, match: np.ndarray, cm: np.ndarray, n_c: int) -> Dict[str, np.ndarray]:
    """Coarse CSR graph (oracle.c: oracle_contract, P12.s26-28, P20.s0-26)."""
    lib = _load()
    g = as_numpy_graph(g)
    match = _np32(match)
    cm = _np32(cm)
    nnz = g["nnz"]
    cadjp = np.zeros(n_c + 1, dtype=np.int32)
    cadjncy = np.empty(max(nnz, 1), dtype=np.int32)
    cadjwgt = np.empty(max(nnz, 1), dtype=np.int32)
    cvwgt = np.empty(max(n_c, 1), dtype=np.int32)
    cnnz = lib.oracle_contract(g["n"], _p(g["adjp"]), _p(g["adjncy"]), _p(g["adjwgt"]),
                               _p(g["vwgt"]), _p(match), _p(cm), n_c, _p(cadjp),
                               _p(cadjncy), _p(cadjwgt), _p(cvwgt))
    if cnnz < 0:
        raise OverflowError("oracle_contract: coarse weight exceeds int32")
    return {"n": n_c, "nnz": int(cnnz), "adjp": cadjp, "adjncy": cadjncy[:cnnz].copy(),
            "adjwgt": cadjwgt[:cnnz].copy(), "vwgt": cvwgt[:n_c].copy()}


STOP_THRESHOLD = 1   # n <= threshold reached
STOP_STALL = 2       # level shrank by less than (100 - stall_ratio_pct) %
STOP_MAX_LEVELS = 3  # max_levels reached


def coarsen_to(g: Dict, threshold: int, stall_ratio_pct: int = 95, max_levels: int = 64,
               max_rounds: int = 0, tie_seed: int = 0) -> List[Dict]:
    """Level loop (P10.s16, P20.s27-31, P12.s30; readings R12, R13).

    while n > threshold and levels < max_levels:
        M = match_level(G); (CM, n_c) = cmap(M); Gc = contract(G, M, CM)
        keep (M, CM, Gc, rounds)                         (pointer arrays, P20.s27)
        stop after this level if 100*n_c > stall_ratio_pct*n   (Metis-style stall, P12.s30)
        G = Gc
    Returns the list of levels; each level dict holds n, nnz, match, cmap, rounds,
    maximal, coarse (CSR dict), stop_reason (0 = continue).
    """
    levels: List[Dict] = []
    cur = as_numpy_graph(g)
    while cur["n"] > threshold and len(levels) < max_levels:
        m, rounds, maximal = match_level(cur, max_rounds, tie_seed)
        cm, n_c = cmap(m)
        coarse = contract(cur, m, cm, n_c)
        stall = 100 * n_c > stall_ratio_pct * cur["n"]
        lvl = {"n": cur["n"], "nnz": cur["nnz"], "match": m, "cmap": cm, "n_coarse": n_c,
               "rounds": rounds, "maximal": maximal, "coarse": coarse, "stop_reason": 0}
        levels.append(lvl)
        cur = coarse
        if stall:
            lvl["stop_reason"] = STOP_STALL
            break
    if levels and levels[-1]["stop_reason"] == 0:
        levels[-1]["stop_reason"] = STOP_THRESHOLD if cur["n"] <= threshold else STOP_MAX_LEVELS
    return levels


def refine(g: Dict, part, nparts: int, imbalance_pct: int = 3, max_passes: int = 8):
    """Refinement of un-coarsening (oracle.c: oracle_refine; P22.s1-22, reading R18).
    Returns (part int32[n], moves, passes)."""
    lib = _load()
    g = as_numpy_graph(g)
    p = _np32(part).copy()
    moves, passes = ctypes.c_int32(0), ctypes.c_int32(0)
    st = lib.oracle_refine(g["n"], _p(g["adjp"]), _p(g["adjncy"]), _p(g["adjwgt"]), _p(g["vwgt"]), int(nparts),
                           int(imbalance_pct), int(max_passes), _p(p), ctypes.byref(moves), ctypes.byref(passes))
    if st != 0:
        raise ValueError("oracle_refine: bad arguments (labels outside [0, nparts)?)")
    return p, int(moves.value), int(passes.value)


def uncoarsen(g0: Dict, levels: List[Dict], part_coarse, nparts: int, imbalance_pct: int = 3,
              max_passes: int = 8):
    """Un-coarsening (P12.s41-46; P20.s41-P22.s22): from the coarsest graph down to level 0,
    project one level (part_l[u] = part_{l+1}[CM_l[u]]) then refine on that level's fine
    graph.  Returns (part of level 0, total moves)."""
    part = np.asarray(part_coarse, dtype=np.int32)
    total = 0
    for l in range(len(levels) - 1, -1, -1):
        part = project(levels, part, from_level=l, to_level=l)
        fine = g0 if l == 0 else levels[l - 1]["coarse"]
        part, mv, _ = refine(fine, part, nparts, imbalance_pct, max_passes)
        total += mv
    return part, total


def project(levels: List[Dict], part_coarse, from_level: Optional[int] = None, to_level: int = 0) -> np.ndarray:
    """Projection of un-coarsening (P12: "the coarser graph is projected back to the finer
    graph by transferring the partition assignment of each vertex to the corresponding
    vertices in the finer graph"; P20-P22: "each thread specify the partition labels of
    the projected vertices in the finer graph by considering the CM array").

    part_coarse labels the coarse graph produced by level `from_level` (default: the last
    level, i.e. the coarsest graph).  Level by level, finest last:
        part_l[u] = part_{l+1}[CM_l[u]]      for l = from_level, ..., to_level
    Returns the labels of level `to_level`'s fine graph.  Plain numpy gathers, one level at
    a time in the paper's order (coarse to fine).
    """
    if from_level is None:
        from_level = len(levels) - 1
    part = np.asarray(part_coarse, dtype=np.int64)
    for l in range(from_level, to_level - 1, -1):
        cm = np.asarray(levels[l]["cmap"], dtype=np.int64)
        assert len(part) == levels[l]["n_coarse"]
        part = part[cm]
    return part.astype(np.int32)
