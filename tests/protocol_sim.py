"""Sequential simulations of the GPU kernels' protocols (test infrastructure).

These re-state, in plain Python, the phase structure the CUDA kernels use so
that the protocol itself -- fused commit_k + propose_{k+1} rounds over double-buffered
proposals, lazy rescans, the "free after round k" test, the round counting -- can be checked
against the oracle on the CPU.  Concurrency inside a phase is modelled by processing the
vertices of a phase in a random order while the writes of that phase (M, and NONE into the
read buffer for dying vertices) become visible immediately, which is the most adversarial
legal interleaving for the reads the kernel performs.
"""
from __future__ import annotations

import numpy as np

FREE = -1
NONE = -1


def _key(w, v):
    return (int(w) << 32) | (0xFFFFFFFF - int(v))


def simulate_match(adjp, adjncy, adjwgt, seed=0, max_rounds=0, use_cache=True):
    rng = np.random.default_rng(seed)
    n = len(adjp) - 1
    M = np.full(n, FREE, dtype=np.int64)
    P = [np.full(n, 123456789, dtype=np.int64), np.full(n, 987654321, dtype=np.int64)]  # garbage
    S = np.full(n, NONE, dtype=np.int64)  # cached second-heaviest neighbour of the last scan

    def vert(k):
        return NONE if k == 0 else 0xFFFFFFFF - (k & 0xFFFFFFFF)

    # phase 0: round-1 proposals (top-2) of every vertex
    for u in rng.permutation(n):
        keys = sorted((_key(adjwgt[j], adjncy[j]) for j in range(adjp[u], adjp[u + 1])), reverse=True)
        best = keys[0] if keys else 0
        second = keys[1] if len(keys) > 1 else 0
        p = vert(best)
        P[1][u] = p
        S[u] = vert(second)
        if p == NONE:
            P[0][u] = NONE
    live = [u for u in range(n) if P[1][u] != NONE]
    rounds = 0
    maximal = False
    k = 1
    while True:
        Pk, Pn = P[k & 1], P[(k + 1) & 1]
        made = 0
        nxt = []

        def free_after(x):
            # P-only test: a vertex matched in any round <= k has
            # P_k[P_k[x]] == x (matched vertices keep their partner in both buffers); a dead
            # vertex (P = NONE) never neighbours a vertex that still rescans.  M is not read.
            px = Pk[x]
            free = not (px >= 0 and Pk[px] == x)
            # the test the M array would give (M written immediately in this simulation)
            assert free == (M[x] == FREE and not (px >= 0 and Pk[px] == x)), (k, x)
            return free

        for u in rng.permutation(live) if live else []:
            p = Pk[u]
            if p == NONE:
                continue
            q = Pk[p]
            if q == u:
                M[u] = p
                Pn[u] = p
                made += 1
            elif not (q >= 0 and Pk[q] == p):
                Pn[u] = p
                nxt.append(u)
            elif use_cache and S[u] != NONE and free_after(S[u]):
                Pn[u] = S[u]
                S[u] = NONE
                nxt.append(u)
            else:
                keys = sorted((_key(adjwgt[j], adjncy[j]) for j in range(adjp[u], adjp[u + 1])
                               if free_after(adjncy[j])), reverse=True)
                b = vert(keys[0]) if keys else NONE
                S[u] = vert(keys[1]) if len(keys) > 1 else NONE
                Pn[u] = b
                if b == NONE:
                    Pk[u] = NONE
                else:
                    nxt.append(u)
        if made > 0:
            rounds += 1
        live = nxt
        if not live:
            maximal = True
            break
        if max_rounds and rounds >= max_rounds:
            break
        k += 1
    for u in range(n):
        if M[u] == FREE:
            M[u] = u
    return M, rounds, maximal
