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

/*
 * Refinement of un-coarsening (P22.s1-22), written out step by step; reading R18 of
 * DESIGN.md §2 fixes what the paper leaves open (gains from the labels at the start of an
 * iteration, ties to the lower partition id, requests explored in (gain desc, vertex asc)
 * order, the integer balance bounds).
 *
 *   W = sum vwgt;  max_w = ceil(W (100 + imb) / (100 k));  min_w = floor(W (100 - imb) / (100 k))
 *   (3 % imbalance in the paper's experiments, P22.s35).
 *   pass = two iterations, dir = 0 (moves to a HIGHER partition id only) then dir = 1 (to a
 *   LOWER one): the ordering method that forbids concurrent exchanges between two
 *   neighbouring partitions (P22.s8-10).  One iteration:
 *     request  (first kernel, P22.s4-7): every boundary vertex v (a neighbour in another
 *              partition) of partition s takes the destination d of its neighbours' partitions,
 *              in the iteration's direction, with the largest gain
 *                 gain(d) = w(v, d) - w(v, s)      (w(v, X) = sum of v's edge weights into X)
 *              if gain > 0 ("maximum reduction of the edge cut"; ties: lower d), the source
 *              stays >= min_w without v and the destination stays <= max_w with v
 *              ("does not underweight the source or overweight the destination").  The
 *              request (v, gain) goes to d's buffer (P22.s11-15).
 *     explore  (P22.s16-19): per destination d, its requests sorted by gain (descending;
 *              equal gains: lower vertex id first) are accepted in that order while
 *              pw[d] + vwgt[v] <= max_w, pw[d] growing with every accepted move.
 *     apply:   the accepted vertices change partition (all at once).
 *   A pass that moves nothing ends the refinement early (P22.s20-21); at most max_passes.
 * part[] is updated in place.  Returns 0, or -1 on a bad argument.
 */
typedef struct { int32_t v; int32_t gain; } oracle_req;

static int oracle_req_cmp(const void *a, const void *b)
{
    const oracle_req *x = (const oracle_req *)a, *y = (const oracle_req *)b;
    if (x->gain != y->gain) return x->gain > y->gain ? -1 : 1;   /* gain descending */
    return (x->v > y->v) - (x->v < y->v);                          /* then vertex id  */
}

int oracle_refine(int32_t n, const int32_t *adjp, const int32_t *adjncy, const int32_t *adjwgt,
                  const int32_t *vwgt, int32_t k, int32_t imbalance_pct, int32_t max_passes,
                  int32_t *part, int32_t *moves_out, int32_t *passes_out)
{
    int64_t W = 0, maxw, minw, *pw, *conn;
    int32_t *dest, *gainv, v, pass, moves = 0, passes = 0;
    oracle_req *req;
    if (k < 1 || imbalance_pct < 0 || max_passes < 0) return -1;
    for (v = 0; v < n; ++v) {
        if (part[v] < 0 || part[v] >= k) return -1;
        W += vwgt[v];
    }
    maxw = (W * (100 + imbalance_pct) + 100LL * k - 1) / (100LL * k);
    minw = (W * (100 - imbalance_pct)) / (100LL * k);
    pw = (int64_t *)calloc((size_t)k, sizeof(int64_t));
    conn = (int64_t *)calloc((size_t)k, sizeof(int64_t));
    dest = (int32_t *)malloc(sizeof(int32_t) * (size_t)(n > 0 ? n : 1));
    gainv = (int32_t *)malloc(sizeof(int32_t) * (size_t)(n > 0 ? n : 1));
    req = (oracle_req *)malloc(sizeof(oracle_req) * (size_t)(n > 0 ? n : 1));
    for (v = 0; v < n; ++v) pw[part[v]] += vwgt[v];

    for (pass = 0; pass < max_passes; ++pass) {
        int32_t pass_moves = 0, dir;
        for (dir = 0; dir < 2; ++dir) {
            int32_t d, j;
            /* request */
            for (v = 0; v < n; ++v) {
                int32_t s = part[v], boundary = 0, best = -1;
                int64_t bestgain = 0;
                dest[v] = -1;
                for (j = adjp[v]; j < adjp[v + 1]; ++j) {
                    int32_t p = part[adjncy[j]];
                    conn[p] += adjwgt[j];
                    if (p != s) boundary = 1;
                }
                if (boundary) {
                    for (j = adjp[v]; j < adjp[v + 1]; ++j) {
                        int64_t g;
                        d = part[adjncy[j]];
                        if (d == s || (dir == 0 ? d < s : d > s)) continue;
                        g = conn[d] - conn[s];
                        if (g > 0 && (best < 0 || g > bestgain || (g == bestgain && d < best))) {
                            best = d;
                            bestgain = g;
                        }
                    }
                    if (best >= 0 && pw[s] - vwgt[v] >= minw && pw[best] + vwgt[v] <= maxw) {
                        dest[v] = best;
                        gainv[v] = (int32_t)bestgain;
                    }
                }
                for (j = adjp[v]; j < adjp[v + 1]; ++j) conn[part[adjncy[j]]] = 0;
            }
            /* explore, one destination partition at a time */
            for (d = 0; d < k; ++d) {
                int32_t m = 0, i;
                int64_t cur = pw[d];
                for (v = 0; v < n; ++v)
                    if (dest[v] == d) { req[m].v = v; req[m].gain = gainv[v]; ++m; }
                qsort(req, (size_t)m, sizeof(oracle_req), oracle_req_cmp);
                for (i = 0; i < m; ++i) {
                    int32_t u = req[i].v;
                    if (cur + vwgt[u] <= maxw) cur += vwgt[u];
                    else dest[u] = -1;                       /* rejected */
                }
            }
            /* apply */
            for (v = 0; v < n; ++v)
                if (dest[v] >= 0) {
                    pw[part[v]] -= vwgt[v];
                    pw[dest[v]] += vwgt[v];
                    part[v] = dest[v];
                    ++pass_moves;
                }
        }
        moves += pass_moves;
        ++passes;
        if (pass_moves == 0) break;
    }
    free(pw);
    free(conn);
    free(dest);
    free(gainv);
    free(req);
    if (moves_out) *moves_out = moves;
    if (passes_out) *passes_out = passes;
    return 0;
}
