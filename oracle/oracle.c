/*
 * oracle.c -- TEST INFRASTRUCTURE ONLY.  Plain, slow, single-threaded C reference of the
 * GP-metis coarsening level (Goodarzi, Burtscher, Goswami, IPDPS-W 2016; PAPER.md).
 *
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference legs
 * may load this file's library.  The product (paper_conf_ipps_goodarzibg16_b200/) never
 * links, imports or calls it, and it shares no code, header, table or helper with the
 * CUDA path.
 *
 * Citations: "P<line>.s<k>" = /root/reference/PAPER.md line <line>, sentence <k>
 * (sentence split rule in SURVEY.md §0).  Readings of garbled/silent passages are the
 * numbered R-items of DESIGN.md §2.
 *
 * Pinning (tests/test_oracle_*.py, -m "not gpu"):
 *   oracle_match_level : hand-worked golden graphs (tests/golden/), equality with the
 *                        textbook sequential greedy matching under the strict edge order
 *                        (independent Python code), brute-force maximality and the 1/2
 *                        weight bound on <= 10 vertices, the closed form of config C1.
 *   oracle_cmap        : golden graphs; permutation/onto/monotone properties.
 *   oracle_contract    : golden graphs; off-diagonal of P^T A P and P^T vwgt computed with
 *                        scipy.sparse (a library primitive, not this code); weight sums.
 * No function here is "parity unpinned".
 *
 * Integer widths (R14): ids, offsets and weights are int32; sums are formed in int64 and
 * an overflow of int32 is reported as an error (-2).
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#define ORACLE_FREE (-1)   /* vertex not yet matched                              */
#define ORACLE_NONE (-1)   /* no proposal: no free neighbour                      */

/*
 * Heavy-edge preference of vertex u between two neighbours (P12.s23, P18.s7): the heavier
 * edge wins; on equal weight the lower vertex id wins (north_star tie rule, R3).
 * Returns nonzero iff (w1, v1) is preferred over (w2, v2).
 */
static int oracle_prefers(int32_t w1, int32_t v1, int32_t w2, int32_t v2)
{
    if (w1 != w2) return w1 > w2;
    return v1 < v2;
}

/*
 * RM tie priority (reading R17 of DESIGN.md §2 for P18.s8: "If all the edges have the same
 * weight, a random matching (RM) ... where each vertex chooses one of its unmatched
 * vertices randomly").  The random choice is made deterministic by a seeded counter-based
 * priority: h_s(v) = lowbias32(v XOR s), all arithmetic mod 2^32:
 *   x ^= x >> 16;  x *= 0x7feb352d;  x ^= x >> 15;  x *= 0x846ca68b;  x ^= x >> 16.
 * Exported so that the tests can pin it against an independent Python transcription.
 */
uint32_t oracle_tie_hash(uint32_t v, uint32_t s)
{
    uint32_t x = v ^ s;
    x ^= x >> 16;
    x *= 0x7feb352du;
    x ^= x >> 15;
    x *= 0x846ca68bu;
    x ^= x >> 16;
    return x;
}

/*
 * Preference under a tie seed s != 0: the heavier edge wins; on equal weight the lower
 * h_s(v) wins.  s == 0 is oracle_prefers (north_star rule).
 */
static int oracle_prefers_seeded(int32_t w1, int32_t v1, int32_t w2, int32_t v2, uint32_t s)
{
    if (s == 0) return oracle_prefers(w1, v1, w2, v2);
    if (w1 != w2) return w1 > w2;
    return oracle_tie_hash((uint32_t)v1, s) < oracle_tie_hash((uint32_t)v2, s);
}

/*
 * One matching level (P16.s23-25, P18.s6-13 and north_star's pinned rule, R1-R4):
 *
 *   M[u] = FREE for all u; rounds = 0
 *   repeat:
 *     for every FREE u: P[u] = heaviest edge (u,v) with v FREE, ties -> lower v;
 *                       P[u] = NONE if u has no FREE neighbour          (HEM, P18.s7-8)
 *     if no FREE u has P[u] != NONE: stop   (no edge joins two free vertices: maximal,
 *                                            P12.s21)
 *     if max_rounds > 0 and rounds == max_rounds: stop (cap; result non-maximal)
 *     for every FREE u with P[u] != NONE: if P[P[u]] == u then M'[u] = P[u]
 *                                           (handshake; replaces the conflict kernel's
 *                                            "M[u]=v and M[v]!=u" test, P18.s10-12)
 *     M = M'; rounds += 1
 *   leftover: M[u] = u for every u still FREE ("matches vertex to itself", P18.s12-13)
 *
 * Every round recomputes P for every free vertex (no lazy rescans: slow and literal).
 * rounds_out = number of rounds that created >= 1 match (R4).
 * maximal_out = 1 iff the loop ended because no free vertex had a free neighbour.
 * Returns 0 on success, -1 if a round with a proposing vertex created no match (the
 * termination lemma of DESIGN.md §2 says this cannot happen; the tests assert it).
 */
int oracle_match_level_seeded(int32_t n, const int32_t *adjp, const int32_t *adjncy,
                              const int32_t *adjwgt, int32_t max_rounds, uint32_t tie_seed,
                              int32_t *match, int32_t *rounds_out, int32_t *maximal_out)
{
    int32_t *P = (int32_t *)malloc(sizeof(int32_t) * (size_t)(n > 0 ? n : 1));
    int32_t *Mn = (int32_t *)malloc(sizeof(int32_t) * (size_t)(n > 0 ? n : 1));
    int32_t rounds = 0;
    int32_t maximal = 0;
    int status = 0;
    int32_t u;

    for (u = 0; u < n; ++u) match[u] = ORACLE_FREE;

    for (;;) {
        int64_t proposing = 0;
        int64_t made = 0;

        /* proposal step: heaviest free neighbour of every free vertex */
        for (u = 0; u < n; ++u) {
            int32_t best_v = ORACLE_NONE, best_w = 0;
            int32_t j;
            P[u] = ORACLE_NONE;
            if (match[u] != ORACLE_FREE) continue;
            for (j = adjp[u]; j < adjp[u + 1]; ++j) {
                int32_t v = adjncy[j];
                int32_t w = adjwgt[j];
                if (match[v] != ORACLE_FREE) continue;
                if (best_v == ORACLE_NONE || oracle_prefers_seeded(w, v, best_w, best_v, tie_seed)) {
                    best_v = v;
                    best_w = w;
                }
            }
            P[u] = best_v;
            if (best_v != ORACLE_NONE) ++proposing;
        }
        if (proposing == 0) { maximal = 1; break; }
        if (max_rounds > 0 && rounds == max_rounds) break;

        /* handshake step: synchronous, reads P only */
        memcpy(Mn, match, sizeof(int32_t) * (size_t)n);
        for (u = 0; u < n; ++u) {
            if (match[u] != ORACLE_FREE || P[u] == ORACLE_NONE) continue;
            if (P[P[u]] == u) { Mn[u] = P[u]; ++made; }
        }
        memcpy(match, Mn, sizeof(int32_t) * (size_t)n);
        if (made == 0) { status = -1; break; }
        rounds += 1;
    }

    /* leftover pass (P18.s12-13): unmatched vertices are matched to themselves */
    for (u = 0; u < n; ++u)
        if (match[u] == ORACLE_FREE) match[u] = u;

    if (rounds_out) *rounds_out = rounds;
    if (maximal_out) *maximal_out = maximal;
    free(P);
    free(Mn);
    return status;
}

/* The north_star rule: lower id wins ties (tie seed 0). */
int oracle_match_level(int32_t n, const int32_t *adjp, const int32_t *adjncy,
                       const int32_t *adjwgt, int32_t max_rounds,
                       int32_t *match, int32_t *rounds_out, int32_t *maximal_out)
{
    return oracle_match_level_seeded(n, adjp, adjncy, adjwgt, max_rounds, 0u,
                                     match, rounds_out, maximal_out);
}

/*
 * Mapping array CM (P18.s16-27), the four steps written out literally:
 *   1. CM[u] = (u <= M[u]) ? 1 : 0                           (P18.s17-18, R7)
 *   2. inclusive prefix sum of CM; the last entry is n_c     (P18.s20-22)
 *   3. subtract one from every entry                         (P18.s23-24)
 *   4. if (u > M[u]) CM[u] = CM[M[u]]                        (P18.s25-26, R7)
 * Returns n_c.
 */
int32_t oracle_cmap(int32_t n, const int32_t *match, int32_t *cmap)
{
    int32_t u, n_c = 0;
    for (u = 0; u < n; ++u) cmap[u] = (u <= match[u]) ? 1 : 0;           /* step 1 */
    for (u = 1; u < n; ++u) cmap[u] += cmap[u - 1];                       /* step 2 */
    if (n > 0) n_c = cmap[n - 1];
    for (u = 0; u < n; ++u) cmap[u] -= 1;                                 /* step 3 */
    for (u = 0; u < n; ++u)                                               /* step 4 */
        if (u > match[u]) cmap[u] = cmap[match[u]];
    return n_c;
}

typedef struct { int32_t key; int32_t w; } oracle_pair;

static int oracle_pair_cmp(const void *a, const void *b)
{
    int32_t x = ((const oracle_pair *)a)->key, y = ((const oracle_pair *)b)->key;
    return (x > y) - (x < y);
}

/*
 * Contraction (P12.s26-28, P20.s0-26), the paper's first merge approach (P20.s16): for the
 * coarse vertex c with leader u (u <= M[u]) and partner v = M[u]:
 *   cvwgt[c] = vwgt[u] + (v != u ? vwgt[v] : 0)                         (P12.s27)
 *   the neighbour lists of u and v are merged, mapped through CM, sorted by quicksort and
 *   repeated coarse neighbours removed with their weights summed (P20.s16, P12.s28, R8);
 *   the collapsed edge (coarse neighbour == c) is dropped (R9); rows are emitted in
 *   ascending coarse id (R10); cadjp is the standard CSR offset array (R11).
 * Caller allocates cadjp[n_c+1], cadjncy[nnz], cadjwgt[nnz], cvwgt[n_c] (nnz = adjp[n] is
 * an upper bound of cnnz, P20.s5-11).
 * Returns cnnz, or -2 if a coarse weight overflows int32.
 */
int64_t oracle_contract(int32_t n, const int32_t *adjp, const int32_t *adjncy,
                        const int32_t *adjwgt, const int32_t *vwgt,
                        const int32_t *match, const int32_t *cmap, int32_t n_c,
                        int32_t *cadjp, int32_t *cadjncy, int32_t *cadjwgt, int32_t *cvwgt)
{
    int32_t maxdeg = 0, u;
    int64_t cnnz = 0;
    oracle_pair *buf;
    for (u = 0; u < n; ++u)
        if (adjp[u + 1] - adjp[u] > maxdeg) maxdeg = adjp[u + 1] - adjp[u];
    buf = (oracle_pair *)malloc(sizeof(oracle_pair) * (size_t)(2 * maxdeg + 1));

    cadjp[0] = 0;
    for (u = 0; u < n; ++u) {
        int32_t v = match[u];
        int32_t c, len = 0, side, i;
        int64_t vw;
        if (u > v) continue;                       /* only leaders create coarse vertices */
        c = cmap[u];
        vw = (int64_t)vwgt[u] + (v != u ? (int64_t)vwgt[v] : 0);
        if (vw > INT32_MAX) { free(buf); return -2; }
        cvwgt[c] = (int32_t)vw;
        for (side = 0; side < (v != u ? 2 : 1); ++side) {
            int32_t y = side == 0 ? u : v, j;
            for (j = adjp[y]; j < adjp[y + 1]; ++j) {
                buf[len].key = cmap[adjncy[j]];
                buf[len].w = adjwgt[j];
                ++len;
            }
        }
        qsort(buf, (size_t)len, sizeof(oracle_pair), oracle_pair_cmp);
        for (i = 0; i < len;) {
            int32_t key = buf[i].key;
            int64_t s = 0;
            while (i < len && buf[i].key == key) { s += buf[i].w; ++i; }
            if (key == c) continue;                /* collapsed edge: no self-loop (R9) */
            if (s > INT32_MAX) { free(buf); return -2; }
            cadjncy[cnnz] = key;
            cadjwgt[cnnz] = (int32_t)s;
            ++cnnz;
        }
        cadjp[c + 1] = (int32_t)cnnz;
    }
    free(buf);
    return cnnz;
}
