"""Plain-Python restatement of the SHARDED coarsening protocol (csrc/dist.cu), one process per
rank, exchanging through torch.distributed (test infrastructure; gloo on the CPU).

Each rank owns the contiguous global ids [vbase, vbase + nloc) with their CSR rows (global
column ids) and keeps globally indexed P / M / CM arrays whose foreign entries are a ghost
cache filled only by the exchanges, exactly as the CUDA driver does:

  matching   phase 0 -> all-gather of boundary records (v, P[v], P[P[v]] if P[v] is the
             owner's else -2) + {live, made} -> round k: commit (P_k[P_k[u]] == u) and the
             proposals of round k+1 over "x free after round k" = not (P_k[P_k[x]] == x) ->
             all-gather -> ... until the global live count is 0; leftover self-matches.
  contract   leader counts all-gathered -> rank offsets of the coarse ids; local CM; boundary
             (v, M[v], CM[v] or -1) all-gathered, resolved in two passes; rows of non-leaders
             whose leader is remote sent to the leader's rank with CM of every neighbour;
             merged rows sorted by coarse id, weights summed, collapsed edge dropped.

Nothing here shares code with oracle/ or the CUDA path; the test compares the gathered
pieces with the oracle.
"""
from __future__ import annotations

from typing import Dict, List

import numpy as np
import torch
import torch.distributed as dist

NONE = -1
NO_PP = -2


def _allgather_rows(rows: np.ndarray, width: int) -> List[np.ndarray]:
    """all-gather of a [k, width] int64 array per rank (padded to the max k)."""
    G = dist.get_world_size()
    k = torch.tensor([rows.shape[0]], dtype=torch.int64)
    ks = [torch.zeros(1, dtype=torch.int64) for _ in range(G)]
    dist.all_gather(ks, k)
    kmax = max(int(x) for x in ks)
    buf = torch.zeros((max(kmax, 1), width), dtype=torch.int64)
    if rows.shape[0]:
        buf[: rows.shape[0]] = torch.from_numpy(rows.astype(np.int64))
    outs = [torch.zeros_like(buf) for _ in range(G)]
    dist.all_gather(outs, buf)
    return [o[: int(kk)].numpy() for o, kk in zip(outs, ks)]


def _exchange(send: Dict[int, np.ndarray], width: int) -> Dict[int, np.ndarray]:
    """point-to-point: send[d] goes to rank d; returns what every other rank sent here."""
    G, me = dist.get_world_size(), dist.get_rank()
    counts = torch.zeros(G, dtype=torch.int64)
    for d, a in send.items():
        counts[d] = a.shape[0]
    allc = [torch.zeros(G, dtype=torch.int64) for _ in range(G)]
    dist.all_gather(allc, counts)
    reqs, recv = [], {}
    for d in range(G):
        if d != me and int(counts[d]) > 0:
            reqs.append(dist.isend(torch.from_numpy(send[d].astype(np.int64)).contiguous(), d))
    for s in range(G):
        c = int(allc[s][me])
        if s != me and c > 0:
            t = torch.zeros((c, width), dtype=torch.int64)
            reqs.append(dist.irecv(t, s))
            recv[s] = t
    for r in reqs:
        r.wait()
    return {s: t.numpy() for s, t in recv.items()}


TIE_SEED = 0  # RM tie priority (DESIGN R17); set by coarsen_to


def _tie(v):
    """Tie priority of v: its id (seed 0) or lowbias32(v ^ seed)."""
    if TIE_SEED == 0:
        return int(v)
    x = (int(v) ^ TIE_SEED) & 0xFFFFFFFF
    x ^= x >> 16
    x = (x * 0x7FEB352D) & 0xFFFFFFFF
    x ^= x >> 15
    x = (x * 0x846CA68B) & 0xFFFFFFFF
    return x ^ (x >> 16)


def _key(w, v):
    return ((int(w) << 32) | (0xFFFFFFFF - _tie(v)), int(v))


def _key_vertex(k):
    return NONE if k == 0 else k[1]


class Shard:
    def __init__(self, n_global, vbase, adjp, adjncy, adjwgt, vwgt, ranges):
        self.N = n_global
        self.vbase = vbase
        self.nloc = len(adjp) - 1
        self.adjp, self.adjncy, self.adjwgt, self.vwgt = adjp, adjncy, adjwgt, vwgt
        self.ranges = ranges  # G + 1

    def local(self, x):
        return self.vbase <= x < self.vbase + self.nloc

    def owner(self, x):
        return int(np.searchsorted(self.ranges, x, side="right") - 1)

    def row(self, u):
        r = u - self.vbase
        return range(self.adjp[r], self.adjp[r + 1])


def shard_of(g: Dict, rank: int, G: int) -> Shard:
    n = len(g["adjp"]) - 1
    ranges = np.array([n * i // G for i in range(G + 1)], dtype=np.int64)
    vb, ve = int(ranges[rank]), int(ranges[rank + 1])
    adjp = np.asarray(g["adjp"], dtype=np.int64)
    a0, a1 = int(adjp[vb]), int(adjp[ve])
    return Shard(n, vb, adjp[vb: ve + 1] - a0, np.asarray(g["adjncy"], dtype=np.int64)[a0:a1],
                 np.asarray(g["adjwgt"], dtype=np.int64)[a0:a1], np.asarray(g["vwgt"], dtype=np.int64)[vb:ve],
                 ranges)


def match_level(sh: Shard, max_rounds: int = 0):
    N = sh.N
    P = [np.full(N, 999999999, dtype=np.int64), np.full(N, 999999999, dtype=np.int64)]  # garbage ghosts
    M = np.full(N, -1, dtype=np.int64)
    loc = range(sh.vbase, sh.vbase + sh.nloc)
    boundary = [u for u in loc if any(not sh.local(int(sh.adjncy[j])) for j in sh.row(u))]

    def publish(Pb, live, made):
        recs = np.array([[v, Pb[v], Pb[Pb[v]] if Pb[v] >= 0 and sh.local(Pb[v]) else NO_PP] for v in boundary],
                        dtype=np.int64).reshape(-1, 3)
        hdr = np.array([[live, made, 0]], dtype=np.int64)
        parts = _allgather_rows(np.vstack([hdr, recs]), 3)
        me = dist.get_rank()
        for s, part in enumerate(parts):
            if s == me:
                continue
            for v, p, pp in part[1:]:
                Pb[v] = p
                if pp != NO_PP:
                    Pb[p] = pp
        return sum(int(p[0, 0]) for p in parts), any(int(p[0, 1]) for p in parts)

    # phase 0: every vertex free
    for u in loc:
        keys = [_key(sh.adjwgt[j], sh.adjncy[j]) for j in sh.row(u)]
        k = max(keys) if keys else 0
        P[1][u] = _key_vertex(k)
        if P[1][u] == NONE:
            P[0][u] = NONE
    live = [u for u in loc if P[1][u] != NONE]
    publish(P[1], len(live), 0)
    rounds, maximal, k = 0, False, 1
    while True:
        Pk, Pn = P[k & 1], P[(k + 1) & 1]
        made = 0
        nxt = []

        def free_after(x):
            px = Pk[x]
            return not (px >= 0 and Pk[px] == x)

        matched_now = set()
        for u in live:  # commit of round k (reads P_k only)
            if Pk[Pk[u]] == u:
                matched_now.add(u)
        for u in live:
            p = Pk[u]
            if u in matched_now:
                M[u] = p
                Pn[u] = p
                made += 1
                continue
            keys = [_key(sh.adjwgt[j], sh.adjncy[j]) for j in sh.row(u) if free_after(int(sh.adjncy[j]))]
            kk = max(keys) if keys else 0
            b = _key_vertex(kk)
            Pn[u] = b
            if b == NONE:
                Pk[u] = NONE  # dead: NONE in both buffers (after everyone read P_k[u]? see note)
            else:
                nxt.append(u)
        glive, gmade = publish(Pn, len(nxt), made)
        if gmade:
            rounds += 1
        live = nxt
        if glive == 0:
            maximal = True
            break
        if max_rounds and rounds >= max_rounds:
            break
        k += 1
    for u in loc:  # leftover (P18.s12-13)
        if M[u] == -1:
            M[u] = u
    return M, rounds, maximal


def contract_level(sh: Shard, M: np.ndarray):
    G, me = dist.get_world_size(), dist.get_rank()
    loc = range(sh.vbase, sh.vbase + sh.nloc)
    lead = [u for u in loc if u <= M[u]]
    counts = _allgather_rows(np.array([[len(lead)]], dtype=np.int64), 1)
    nlead = [int(c[0, 0]) for c in counts]
    cbase = int(sum(nlead[:me]))
    NC = int(sum(nlead))
    CM = np.full(sh.N, -7, dtype=np.int64)
    for i, u in enumerate(lead):
        CM[u] = cbase + i
        if M[u] != u and sh.local(M[u]):
            CM[M[u]] = cbase + i
    boundary = [u for u in loc if any(not sh.local(int(sh.adjncy[j])) for j in sh.row(u))]
    recs = np.array([[v, M[v], CM[v] if (v <= M[v] or sh.local(M[v])) else -1] for v in boundary],
                    dtype=np.int64).reshape(-1, 3)
    parts = _allgather_rows(recs, 3)
    for s, part in enumerate(parts):  # pass 1: known values
        if s != me:
            for v, m, c in part:
                if c >= 0:
                    CM[v] = c
    for s, part in enumerate(parts):  # pass 2: non-leaders copy their leader's id
        if s != me:
            for v, m, c in part:
                if c < 0:
                    CM[v] = CM[m]
    for u in loc:
        if u > M[u] and not sh.local(M[u]):
            CM[u] = CM[M[u]]
    # ship rows of non-leaders with a remote leader: (leader, x, w, CM[x]) per arc, or a
    # (leader, -1, vwgt, 0) record for the vertex itself
    send: Dict[int, list] = {}
    for u in loc:
        m = int(M[u])
        if u > m and not sh.local(m):
            d = sh.owner(m)
            rows = send.setdefault(d, [])
            rows.append([m, -1, int(sh.vwgt[u - sh.vbase]), 0])
            for j in sh.row(u):
                x = int(sh.adjncy[j])
                rows.append([m, x, int(sh.adjwgt[j]), int(CM[x])])
    got = _exchange({d: np.array(r, dtype=np.int64) for d, r in send.items()}, 4)
    shipped: Dict[int, list] = {}
    shipped_vw: Dict[int, int] = {}
    for s, arr in got.items():
        for l, x, w, cx in arr:
            if x == -1:
                shipped_vw[int(l)] = int(w)
            else:
                CM[x] = cx
                shipped.setdefault(int(l), []).append((int(x), int(w)))
    # merge (P12.s26-28): coarse row c = union of both fine rows by CM, collapsed edge dropped
    adjp, adjncy, adjwgt, vwgt = [0], [], [], []
    for i, u in enumerate(lead):
        c = cbase + i
        m = int(M[u])
        arcs = [(int(sh.adjncy[j]), int(sh.adjwgt[j])) for j in sh.row(u)]
        vw = int(sh.vwgt[u - sh.vbase])
        if m != u:
            if sh.local(m):
                arcs += [(int(sh.adjncy[j]), int(sh.adjwgt[j])) for j in sh.row(m)]
                vw += int(sh.vwgt[m - sh.vbase])
            else:
                arcs += shipped.get(u, [])
                vw += shipped_vw[u]
        acc: Dict[int, int] = {}
        for x, w in arcs:
            cx = int(CM[x])
            if cx != c:
                acc[cx] = acc.get(cx, 0) + w
        for cx in sorted(acc):
            adjncy.append(cx)
            adjwgt.append(acc[cx])
        adjp.append(len(adjncy))
        vwgt.append(vw)
    coarse = Shard(NC, cbase, np.array(adjp, dtype=np.int64), np.array(adjncy, dtype=np.int64),
                   np.array(adjwgt, dtype=np.int64), np.array(vwgt, dtype=np.int64),
                   np.concatenate([[0], np.cumsum(nlead)]).astype(np.int64))
    return CM, coarse


def fold(sh: Shard) -> Shard:
    """Folding (csrc/dist.cu fold): every rank gathers the coarse pieces --
    rows (adjp shifted by the arc base of the rank) | vwgt | adjncy | adjwgt -- and the rest of
    the hierarchy runs on the whole graph.  Here that graph is re-sharded onto rank 0 (the
    piece layout the CUDA driver reports for folded levels: rank 0 owns every vertex)."""
    G, me = dist.get_world_size(), dist.get_rank()
    rows = _allgather_rows(np.stack([sh.adjp[1:] - sh.adjp[:-1], sh.vwgt], axis=1) if sh.nloc else
                           np.zeros((0, 2), dtype=np.int64), 2)
    arcs = _allgather_rows(np.stack([sh.adjncy, sh.adjwgt], axis=1) if len(sh.adjncy) else
                           np.zeros((0, 2), dtype=np.int64), 2)
    deg = np.concatenate([r[:, 0] for r in rows]).astype(np.int64)
    assert len(deg) == sh.N
    adjp = np.concatenate([[0], np.cumsum(deg)]).astype(np.int64)
    vwgt = np.concatenate([r[:, 1] for r in rows]).astype(np.int64)
    adjncy = np.concatenate([a[:, 0] for a in arcs]).astype(np.int64)
    adjwgt = np.concatenate([a[:, 1] for a in arcs]).astype(np.int64)
    ranges = np.array([0] + [sh.N] * G, dtype=np.int64)
    if me == 0:
        return Shard(sh.N, 0, adjp, adjncy, adjwgt, vwgt, ranges)
    e = np.zeros(0, dtype=np.int64)
    return Shard(sh.N, sh.N, np.zeros(1, dtype=np.int64), e, e, e, ranges)


def coarsen_to(sh: Shard, threshold: int, stall_ratio_pct: int = 95, max_levels: int = 64, max_rounds: int = 0,
               tie_seed: int = 0, fold_n: int = 0):
    """Levels of this rank: list of dicts with the rank's slices of M / CM and coarse piece.
    fold_n > 0: fold once a coarse graph has at most fold_n vertices (csrc/dist.cu GP_FOLD_N)."""
    global TIE_SEED
    TIE_SEED = tie_seed & 0xFFFFFFFF
    levels = []
    folded = False
    while sh.N > threshold and len(levels) < max_levels:
        M, rounds, maximal = match_level(sh, max_rounds)
        CM, cg = contract_level(sh, M)
        sl = slice(sh.vbase, sh.vbase + sh.nloc)
        levels.append({"n": sh.N, "rounds": rounds, "maximal": maximal, "match": M[sl].copy(), "cmap": CM[sl].copy(),
                       "n_coarse": cg.N, "coarse": cg})
        stall = 100 * cg.N > stall_ratio_pct * sh.N
        sh = cg
        if stall:
            break
        if fold_n > 0 and not folded and sh.N <= fold_n and sh.N > threshold and len(levels) < max_levels:
            sh = fold(sh)
            folded = True
    return levels
