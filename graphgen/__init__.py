"""Seeded, synthetic input generators shared by the oracle tests and the CUDA path.

This module holds NONE of the method's arithmetic (no matching, no cmap, no
contraction).  It only builds undirected, weighted CSR graphs
``G = (V, E, W_v, W_e)`` (PAPER.md P10.s11) in the paper's CSR layout
``adjp[|V|+1], adjncy[2|E|], adjwgt[2|E|], vwgt[|V|]`` (P16.s17-19), shaped like
the paper's workloads (Table I, P22.s33-37) and BASELINE.json's configs.

Every generator is integer-only and counter-based (splitmix64 of a counter), so
the same call on CPU or CUDA returns bit-identical tensors.  All generators take
a ``device`` argument; the bench generates full-size graphs on the GPU, the CPU
tests generate small ones on the host.  Recipes are stated in DESIGN.md §3.

Hash:    h(s, x) = splitmix64(x XOR splitmix64(s))           (64-bit, wrapping)
Weights: w(u, v) = 1 + (h(2, (min(u,v) << 32) | max(u,v)) >>> 33) mod wmax
         (symmetric by construction; vwgt = 1 everywhere)
"""
from __future__ import annotations

import math
from typing import Dict, Optional

import torch

MASK64 = (1 << 64) - 1
_GOLDEN = 0x9E3779B97F4A7C15
_M1 = 0xBF58476D1CE4E5B9
_M2 = 0x94D049BB133111EB

SEED_STRUCTURE = 1
SEED_WEIGHT = 2
SEED_PERMUTE = 3


def _s64(x: int) -> int:
    """Reinterpret an unsigned 64-bit python int as signed int64."""
    x &= MASK64
    return x - (1 << 64) if x >> 63 else x


def _srl(x: torch.Tensor, k: int) -> torch.Tensor:
    """Logical right shift of int64 tensors holding uint64 bit patterns."""
    return (x >> k) & ((1 << (64 - k)) - 1)


def splitmix64_int(x: int) -> int:
    """Scalar splitmix64 on python ints (used for seeds and by the tests)."""
    z = (x + _GOLDEN) & MASK64
    z = ((z ^ (z >> 30)) * _M1) & MASK64
    z = ((z ^ (z >> 27)) * _M2) & MASK64
    return z ^ (z >> 31)


def splitmix64(x: torch.Tensor) -> torch.Tensor:
    """Vectorised splitmix64 over int64 tensors (uint64 bit patterns, wrapping)."""
    z = x + _s64(_GOLDEN)
    z = (z ^ _srl(z, 30)) * _s64(_M1)
    z = (z ^ _srl(z, 27)) * _s64(_M2)
    return z ^ _srl(z, 31)


def h(s: int, x: torch.Tensor) -> torch.Tensor:
    """Counter-based hash stream ``s`` evaluated at counters ``x`` (int64 bit patterns)."""
    return splitmix64(x ^ _s64(splitmix64_int(s)))


def edge_weights(u: torch.Tensor, v: torch.Tensor, wmax: int = 100,
                 seed: int = SEED_WEIGHT) -> torch.Tensor:
    """Symmetric integer edge weights in [1, wmax] keyed by the unordered pair."""
    lo = torch.minimum(u, v).to(torch.int64)
    hi = torch.maximum(u, v).to(torch.int64)
    r = _srl(h(seed, (lo << 32) | hi), 33)          # 31 uniform bits, non-negative
    return (1 + r % wmax).to(torch.int32)


def csr_from_edges(n: int, u: torch.Tensor, v: torch.Tensor, w: torch.Tensor,
                   name: str = "") -> Dict[str, object]:
    """Build the paper's CSR (P16.s18-19) from unique undirected edges u<v.

    Rows are sorted by neighbour id (any order is valid input; the output of the
    method is order-independent, reading R15).
    """
    dev = u.device
    u = u.to(torch.int64)
    v = v.to(torch.int64)
    src = torch.cat([u, v])
    dst = torch.cat([v, u])
    ww = torch.cat([w, w]).to(torch.int32)
    key = src * n + dst
    key, order = torch.sort(key)
    adjncy = (key % n).to(torch.int32)
    adjwgt = ww[order].contiguous()
    deg = torch.bincount(src, minlength=n) if n > 0 else torch.zeros(0, dtype=torch.int64, device=dev)
    adjp = torch.zeros(n + 1, dtype=torch.int64, device=dev)
    if n > 0:
        adjp[1:] = torch.cumsum(deg, 0)
    assert int(adjp[-1]) < 2**31, "nnz must fit int32"
    return {
        "name": name,
        "n": n,
        "nnz": int(adjncy.numel()),
        "adjp": adjp.to(torch.int32).contiguous(),
        "adjncy": adjncy.contiguous(),
        "adjwgt": adjwgt,
        "vwgt": torch.ones(n, dtype=torch.int32, device=dev),
    }


def shuffle_rows(g: Dict[str, object], seed: int) -> Dict[str, object]:
    """The same graph with every row's neighbours in a seeded pseudo-random order (input
    contract R15: any neighbour order is valid).  Arcs are permuted inside their row by the
    key (row, h(seed, arc index)); weights move with their arcs."""
    adjp = g["adjp"]
    dev = adjp.device
    n = adjp.numel() - 1
    nnz = int(adjp[-1]) if n >= 0 else 0
    out = dict(g)
    if nnz == 0:
        return out
    row = torch.repeat_interleave(torch.arange(n, device=dev, dtype=torch.int64), torch.diff(adjp).to(torch.int64))
    r = _srl(h(7000 + seed, torch.arange(nnz, device=dev, dtype=torch.int64)), 33)  # 31 random bits
    perm = torch.argsort((row << 31) | r)
    out["adjncy"] = g["adjncy"][perm].contiguous()
    out["adjwgt"] = g["adjwgt"][perm].contiguous()
    out["name"] = f"{g.get('name', '')}_shuf{seed}"
    return out


def varied_vwgt(g: Dict[str, object], period: int = 7) -> Dict[str, object]:
    """The same graph with non-unit vertex weights vwgt[u] = 1 + u mod period."""
    n = g["adjp"].numel() - 1
    out = dict(g)
    out["vwgt"] = (1 + torch.arange(n, device=g["adjp"].device, dtype=torch.int64) % period).to(torch.int32)
    return out


def _unique_pairs(u: torch.Tensor, v: torch.Tensor) -> (torch.Tensor, torch.Tensor):
    """Drop self-loops, orient u<v, deduplicate."""
    keep = u != v
    u, v = u[keep], v[keep]
    lo = torch.minimum(u, v)
    hi = torch.maximum(u, v)
    key = torch.unique((lo << 32) | hi)
    return key >> 32, key & 0xFFFFFFFF


# --------------------------------------------------------------------------------------
# configs[0]: 64x64 2D grid, unit weights (C1)
# --------------------------------------------------------------------------------------
def grid2d(rows: int, cols: int, unit: bool = True, wmax: int = 100,
           device: str = "cpu") -> Dict[str, object]:
    """4-neighbour rows x cols lattice, row-major ids (a 2D mesh, Table I analogue)."""
    r = torch.arange(rows, device=device, dtype=torch.int64)
    c = torch.arange(cols, device=device, dtype=torch.int64)
    rr, cc = torch.meshgrid(r, c, indexing="ij")
    ids = rr * cols + cc
    hu = ids[:, :-1].reshape(-1)
    hv = ids[:, 1:].reshape(-1)
    vu = ids[:-1, :].reshape(-1)
    vv = ids[1:, :].reshape(-1)
    u = torch.cat([hu, vu])
    v = torch.cat([hv, vv])
    w = torch.ones_like(u, dtype=torch.int32) if unit else edge_weights(u, v, wmax)
    return csr_from_edges(rows * cols, u, v, w, name=f"grid{rows}x{cols}")


# --------------------------------------------------------------------------------------
# configs[2]: Delaunay-like planar triangulated lattice (C3)
# --------------------------------------------------------------------------------------
def delaunay_like(side: int, wmax: int = 100, device: str = "cpu") -> Dict[str, object]:
    """side x side lattice plus one diagonal per cell chosen by a hash bit.

    Planar triangulation; |E| = 2*side*(side-1) + (side-1)^2; degrees 2..8, avg ~6
    (delaunay_n20 of Table I has avg degree 6.0, P22.s37).  Row-major ids.
    """
    r = torch.arange(side, device=device, dtype=torch.int64)
    rr, cc = torch.meshgrid(r, r, indexing="ij")
    ids = rr * side + cc
    hu, hv = ids[:, :-1].reshape(-1), ids[:, 1:].reshape(-1)
    vu, vv = ids[:-1, :].reshape(-1), ids[1:, :].reshape(-1)
    cell = ids[:-1, :-1].reshape(-1)                   # top-left corner id of each cell
    bit = h(SEED_STRUCTURE, cell) & 1
    du = torch.where(bit == 1, cell, cell + 1)          # (r,c)-(r+1,c+1)  or  (r,c+1)-(r+1,c)
    dv = torch.where(bit == 1, cell + side + 1, cell + side)
    u = torch.cat([hu, vu, du])
    v = torch.cat([hv, vv, dv])
    lo, hi = torch.minimum(u, v), torch.maximum(u, v)
    return csr_from_edges(side * side, lo, hi, edge_weights(lo, hi, wmax), name=f"delaunay_like{side}")


# --------------------------------------------------------------------------------------
# configs[1]: random geometric graph (C2), integer coordinates -> exact on any device
# --------------------------------------------------------------------------------------
RGG_COORD_BITS = 21


def rgg_radius_int(n: int, radius_factor: float = 0.55) -> int:
    """Integer connection radius on the 2^21 x 2^21 coordinate lattice."""
    r = radius_factor * math.sqrt(math.log(n) / n)
    return max(1, int(r * (1 << RGG_COORD_BITS)))


def rgg(n: int, wmax: int = 100, radius_factor: float = 0.55,
        device: str = "cpu") -> Dict[str, object]:
    """Random geometric graph: n points uniform on a 2^21 integer lattice, edge iff
    squared distance < R^2, ids sorted by (cell_y, cell_x, draw index) with cell side R
    (spatial ids like DIMACS10 rgg_n_2_* files).  Average degree ~ pi*0.55^2*ln n.
    """
    i = torch.arange(n, device=device, dtype=torch.int64)
    X = _srl(h(SEED_STRUCTURE, 2 * i), 64 - RGG_COORD_BITS)
    Y = _srl(h(SEED_STRUCTURE, 2 * i + 1), 64 - RGG_COORD_BITS)
    R = rgg_radius_int(n, radius_factor)
    R2 = R * R
    g = ((1 << RGG_COORD_BITS) + R - 1) // R           # cells per side
    cx, cy = X // R, Y // R
    cid = cy * g + cx
    key = cid * n + i
    _, order = torch.sort(key)
    X, Y, cx, cy, cid = X[order], Y[order], cx[order], cy[order], cid[order]   # new id = position
    cnt = torch.bincount(cid, minlength=g * g)
    start = torch.zeros(g * g + 1, dtype=torch.int64, device=device)
    start[1:] = torch.cumsum(cnt, 0)
    us, vs = [], []
    # half-neighbourhood: same cell (j>i), (+1,0), (-1,+1), (0,+1), (+1,+1)
    for dx, dy in ((0, 0), (1, 0), (-1, 1), (0, 1), (1, 1)):
        nx, ny = cx + dx, cy + dy
        ok = (nx >= 0) & (nx < g) & (ny < g)
        src = torch.nonzero(ok).squeeze(1)
        nb = (ny[src] * g + nx[src])
        c = cnt[nb]
        a = torch.repeat_interleave(src, c)
        base = torch.repeat_interleave(start[nb], c)
        off = torch.arange(a.numel(), device=device, dtype=torch.int64)
        grp_start = torch.repeat_interleave(torch.cumsum(c, 0) - c, c)
        b = base + (off - grp_start)
        if dx == 0 and dy == 0:
            m = b > a
            a, b = a[m], b[m]
        ddx = X[a] - X[b]
        ddy = Y[a] - Y[b]
        m = ddx * ddx + ddy * ddy < R2
        us.append(a[m])
        vs.append(b[m])
    u = torch.cat(us)
    v = torch.cat(vs)
    lo, hi = torch.minimum(u, v), torch.maximum(u, v)
    return csr_from_edges(n, lo, hi, edge_weights(lo, hi, wmax), name=f"rgg{n}")


# --------------------------------------------------------------------------------------
# configs[3]: Graph500-style R-MAT (C4)
# --------------------------------------------------------------------------------------
def rmat(scale: int, edge_factor: int = 16, wmax: int = 100, unit: bool = False,
         abcd=(0.57, 0.19, 0.19, 0.05), permute: bool = True,
         device: str = "cpu", chunk: int = 1 << 26) -> Dict[str, object]:
    """R-MAT (a,b,c,d) = (0.57,0.19,0.19,0.05), 2^scale * edge_factor endpoint pairs,
    self-loops dropped, symmetrised, deduplicated, ids permuted Graph500-style."""
    n = 1 << scale
    m = n * edge_factor
    a, b, c, _ = abcd
    t1 = int(a * (1 << 53))
    t2 = int((a + b) * (1 << 53))
    t3 = int((a + b + c) * (1 << 53))
    keys = []
    for e0 in range(0, m, chunk):
        e = torch.arange(e0, min(m, e0 + chunk), device=device, dtype=torch.int64)
        src = torch.zeros_like(e)
        dst = torch.zeros_like(e)
        for bit in range(scale):
            r = _srl(h(SEED_STRUCTURE, e * 64 + bit), 11)
            qi = (r >= t2).to(torch.int64)                       # quadrants (1,0),(1,1)
            qj = ((r >= t1) & (r < t2)) | (r >= t3)              # quadrants (0,1),(1,1)
            src = src * 2 + qi
            dst = dst * 2 + qj.to(torch.int64)
        keep = src != dst
        src, dst = src[keep], dst[keep]
        lo, hi = torch.minimum(src, dst), torch.maximum(src, dst)
        keys.append(torch.unique((lo << 32) | hi))
        del e, src, dst, lo, hi
    key = torch.unique(torch.cat(keys))
    lo, hi = key >> 32, key & 0xFFFFFFFF
    if permute:
        # vertex i -> rank of h(3, i) among all hashes (a seeded bijection)
        hv = h(SEED_PERMUTE, torch.arange(n, device=device, dtype=torch.int64))
        order = torch.sort(hv, stable=True).indices
        pos = torch.empty_like(order)
        pos[order] = torch.arange(n, device=device, dtype=torch.int64)
        lo, hi = pos[lo], pos[hi]
        lo, hi = torch.minimum(lo, hi), torch.maximum(lo, hi)
    w = torch.ones_like(lo, dtype=torch.int32) if unit else edge_weights(lo, hi, wmax)
    return csr_from_edges(n, lo, hi, w, name=f"rmat{scale}")


# --------------------------------------------------------------------------------------
# configs[4]: road-network-like sparse lattice (C5)
# --------------------------------------------------------------------------------------
def road_like(side: int, keep_prob: float = 0.625, wmax: int = 100,
              device: str = "cpu") -> Dict[str, object]:
    """side x side lattice keeping each lattice edge e iff h(1,e)>>>11 < p*2^53.

    Average degree ~ 4p = 2.5 (USA Roads in Table I has 2.42, P22.s37); ~2 % of
    vertices isolated; row-major ids; integer travel-like weights in [1, wmax].
    """
    nh = side * (side - 1)
    nv = (side - 1) * side
    e = torch.arange(nh + nv, device=device, dtype=torch.int64)
    thr = int(keep_prob * (1 << 53))
    keep = _srl(h(SEED_STRUCTURE, e), 11) < thr
    e = e[keep]
    isv = e >= nh
    eh = e
    r_h, c_h = eh // (side - 1), eh % (side - 1)
    ev = e - nh
    r_v, c_v = ev // side, ev % side
    u = torch.where(isv, r_v * side + c_v, r_h * side + c_h)
    v = torch.where(isv, (r_v + 1) * side + c_v, r_h * side + c_h + 1)
    return csr_from_edges(side * side, u, v, edge_weights(u, v, wmax), name=f"road{side}")


# --------------------------------------------------------------------------------------
# small random graphs for tests
# --------------------------------------------------------------------------------------
def random_graph(n: int, m: int, seed: int, wmax: int = 100, device: str = "cpu") -> Dict[str, object]:
    """Erdos-Renyi-like multigraph draw of m pairs (deduplicated, loops dropped)."""
    k = torch.arange(m, device=device, dtype=torch.int64)
    u = _srl(h(1000 + seed, 2 * k), 1) % max(n, 1)
    v = _srl(h(1000 + seed, 2 * k + 1), 1) % max(n, 1)
    lo, hi = _unique_pairs(u, v)
    w = edge_weights(lo, hi, wmax, seed=2000 + seed)
    return csr_from_edges(n, lo, hi, w, name=f"er{n}_{m}_{seed}")


def from_edge_list(n: int, edges, vwgt=None) -> Dict[str, object]:
    """CSR from an explicit python list of (u, v, w) undirected edges (fixtures)."""
    if edges:
        u = torch.tensor([e[0] for e in edges], dtype=torch.int64)
        v = torch.tensor([e[1] for e in edges], dtype=torch.int64)
        w = torch.tensor([e[2] for e in edges], dtype=torch.int32)
    else:
        u = torch.zeros(0, dtype=torch.int64)
        v = torch.zeros(0, dtype=torch.int64)
        w = torch.zeros(0, dtype=torch.int32)
    lo, hi = torch.minimum(u, v), torch.maximum(u, v)
    g = csr_from_edges(n, lo, hi, w, name="fixture")
    if vwgt is not None:
        g["vwgt"] = torch.tensor(vwgt, dtype=torch.int32)
    return g


# --------------------------------------------------------------------------------------
# the five BASELINE.json configs (full size) and reduced-size versions for tests
# --------------------------------------------------------------------------------------
# Weight ranges keep sum(adjwgt) <= INT32_MAX at full size (reading R14): C4 has ~5.2e8 arcs
# (mean weight 2.5 -> ~1.3e9), C5 ~1.7e8 arcs (mean 5.5 -> ~9.2e8).  C2/C3 use [1,100].
C4_WMAX = 4
C5_WMAX = 10

CONFIGS = {
    "C1": dict(desc="64x64 2D grid graph (4,096 vertices, unit weights), coarsen to <=100", threshold=100),
    "C2": dict(desc="random geometric graph rgg n=2^20, avg degree ~13", threshold=100),
    "C3": dict(desc="Delaunay-like planar mesh n=2^22, random integer edge weights", threshold=100),
    "C4": dict(desc="R-MAT scale 24, edge factor 16", threshold=100),
    "C5": dict(desc="road-network-like sparse graph n=2^26, avg degree ~2.5", threshold=100),
}


def make_config(name: str, device: str = "cpu", reduce: int = 0) -> Dict[str, object]:
    """Build config ``name``; ``reduce`` > 0 shrinks it (log2 of n reduced by ``reduce``)."""
    if name == "C1":
        return grid2d(64, 64, unit=True, device=device)
    if name == "C2":
        return rgg(1 << (20 - reduce), device=device)
    if name == "C3":
        return delaunay_like(2048 >> (reduce // 2), device=device)
    if name == "C4":
        return rmat(24 - reduce, 16, wmax=C4_WMAX, device=device)
    if name == "C5":
        return road_like(8192 >> (reduce // 2), wmax=C5_WMAX, device=device)
    raise KeyError(name)
