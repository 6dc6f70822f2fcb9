/*
 * skycube_oracle.c — CPU ORACLE FOR THE MDMC SKYCUBE.  TEST INFRASTRUCTURE ONLY.
 *
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference leg may load,
 * call, link or execute this file.  It shares no code, header, table or constant with the CUDA path
 * (paper_conf_sigmod_boghcsa17_b200/csrc), and the CUDA path never calls it.
 *
 * It is plain, slow and written to be checked against PAPER.md by eye:
 *
 *   Def. 1 (L92, §2.2): p dominates q in subspace 0 < delta < 2^d  iff
 *        (B_{p=q} & delta) != delta  and  (B_{p<=q} & delta) == delta;
 *        p strictly dominates q in delta iff additionally (B_{p=q} & delta) == 0.
 *   Def. 2 (L100): S_delta(P)  = { q in P : no p in P with p dominates q in delta }
 *                    S+_delta(P) = { q in P : no p in P with p strictly dominates q in delta }
 *   Def. 3 (L110):   the skycube maps every 0 < delta < 2^d to S_delta(P).
 *   Bitmasks (L76-84, §2.1): bit i of delta <=> dimension i; bit i of B_{p (op) q} <=> p[i] (op) q[i].
 *   Smaller values are better (footnote 2, L114).  Values are IEEE binary32 compared with < and <=
 *   (reading Q10); no arithmetic is applied to them.
 *
 * Output conventions: membership row of point p = W = max(1, 2^d/32) uint32
 * words; bit delta (word delta>>5, bit delta&31) set <=> p in S_delta(P); bit 0 is always 0.
 * This is the paper's B_{p in S} (L84) unshifted (the paper stores bit delta-1).
 *
 * Two independent algorithms:
 *   oracle_a_*  literal Def. 1-3: per subspace, per point, per competitor (O(2^d n^2 d)).
 *   oracle_b_*  per point p against all of P (not only S+; it does not use the S+ lemma of):
 *               p is dominated in delta  <=>  exists q, exists i in delta:  i in S_qp  and  delta is a
 *               subset of L_qp, where L_qp = B_{q<=p}, S_qp = B_{q<p}.  With G_i = { L_qp : i in S_qp }
 *               and D_i = superset-closure(G_i) (D_i[delta] = OR_{M superset of delta} G_i[M]),
 *               p is dominated in delta  <=>  OR_{i in delta} D_i[delta].
 *               Likewise p is strictly dominated in delta <=> delta is a subset of some S_qp
 *               <=> Ds[delta] with Ds = superset-closure({S_qp}).
 *               This is a restatement of Def. 1 with the same quantifiers, not a different method.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#ifdef _OPENMP
#include <omp.h>
#endif

static inline uint32_t words_per_row(int d) {
    return d >= 5 ? (1u << (d - 5)) : 1u;
}

/* B_{q<=p} and B_{q<p} (L82: bit i of B_{p (op) q} is set iff p[i] (op) q[i]). */
static inline void relation_masks(const float *q, const float *p, int d, uint32_t *le, uint32_t *lt) {
    uint32_t a = 0, b = 0;
    for (int i = 0; i < d; i++) {
        if (q[i] <= p[i]) a |= 1u << i;
        if (q[i] < p[i])  b |= 1u << i;
    }
    *le = a;
    *lt = b;
}

/* Def. 1, literally: q dominates p in delta. */
static inline int dominates(const float *q, const float *p, int d, uint32_t delta) {
    uint32_t le, lt;
    relation_masks(q, p, d, &le, &lt);
    uint32_t eq = le & ~lt;                       /* B_{q=p} */
    return ((eq & delta) != delta) && ((le & delta) == delta);
}

/* Def. 1, strict: q strictly dominates p in delta. */
static inline int strictly_dominates(const float *q, const float *p, int d, uint32_t delta) {
    uint32_t le, lt;
    relation_masks(q, p, d, &le, &lt);
    return (lt & delta) == delta;
}

int oracle_version(void) { return 1; }

int oracle_num_threads(void) {
#ifdef _OPENMP
    return omp_get_max_threads();
#else
    return 1;
#endif
}

/* ---------------------------------------------------------------------------------------------
 * Oracle A — literal (Def. 2 and Def. 3).
 *   rows:     [n][W] out, membership (p in S_delta) per the conventions above.
 *   ext_rows: [n][W] out or NULL, extended-skyline membership (p in S+_delta).
 * ------------------------------------------------------------------------------------------- */
int oracle_a_rows(const float *pts, int64_t n, int d, uint32_t *rows, uint32_t *ext_rows) {
    if (d < 1 || d > 16 || n < 0) return 1;
    const uint32_t W = words_per_row(d);
    const uint32_t full = (1u << d) - 1u;
    memset(rows, 0, sizeof(uint32_t) * (size_t)n * W);
    if (ext_rows) memset(ext_rows, 0, sizeof(uint32_t) * (size_t)n * W);
    #pragma omp parallel for schedule(dynamic, 1)
    for (int64_t p = 0; p < n; p++) {
        const float *pp = pts + (size_t)p * d;
        for (uint32_t delta = 1; delta <= full; delta++) {
            int dominated = 0, sdominated = 0;
            for (int64_t q = 0; q < n; q++) {
                if (q == p) continue;                          /* "a distinct point" (L88) */
                const float *qq = pts + (size_t)q * d;
                if (!dominated && dominates(qq, pp, d, delta)) dominated = 1;
                if (!sdominated && strictly_dominates(qq, pp, d, delta)) sdominated = 1;
                if (dominated && (sdominated || !ext_rows)) break;
            }
            if (!dominated) rows[(size_t)p * W + (delta >> 5)] |= 1u << (delta & 31);
            if (ext_rows && !sdominated) ext_rows[(size_t)p * W + (delta >> 5)] |= 1u << (delta & 31);
        }
    }
    return 0;
}

/* Oracle A on selected (point, subspace) cells: out[k] = 1 iff pids[k] in S_{deltas[k]}(P).
 * Used for sampled parity at full sizes ("outputs the oracle can compute one by one"). */
int oracle_a_cells(const float *pts, int64_t n, int d, const int64_t *pids, const uint32_t *deltas,
                   int64_t ncells, uint8_t *out) {
    if (d < 1 || d > 16) return 1;
    #pragma omp parallel for schedule(dynamic, 16)
    for (int64_t k = 0; k < ncells; k++) {
        const int64_t p = pids[k];
        const uint32_t delta = deltas[k];
        const float *pp = pts + (size_t)p * d;
        int dominated = 0;
        for (int64_t q = 0; q < n && !dominated; q++) {
            if (q == p) continue;
            if (dominates(pts + (size_t)q * d, pp, d, delta)) dominated = 1;
        }
        out[k] = (uint8_t)!dominated;
    }
    return 0;
}

/* S+(P) of Alg. 3 line 2 (L320): ext[p] = 1 iff no q strictly dominates p in the full space. */
int oracle_ext_full(const float *pts, int64_t n, int d, uint8_t *ext) {
    if (d < 1 || d > 16) return 1;
    const uint32_t full = (1u << d) - 1u;
    #pragma omp parallel for schedule(dynamic, 64)
    for (int64_t p = 0; p < n; p++) {
        const float *pp = pts + (size_t)p * d;
        int sd = 0;
        for (int64_t q = 0; q < n && !sd; q++)
            if (q != p && strictly_dominates(pts + (size_t)q * d, pp, d, full)) sd = 1;
        ext[p] = (uint8_t)!sd;
    }
    return 0;
}

/* ---------------------------------------------------------------------------------------------
 * Oracle B — per point p against every q in P, then superset closures.
 * ------------------------------------------------------------------------------------------- */

/* X[delta] := OR over all M that are supersets of delta of X[M] (one pass per dimension). */
static void superset_closure(uint8_t *X, int d) {
    const uint32_t size = 1u << d;
    for (int j = 0; j < d; j++)
        for (uint32_t delta = 0; delta < size; delta++)
            if (!(delta & (1u << j))) X[delta] |= X[delta | (1u << j)];
}

/* Rows for the points pids[0..np) (all of P when pids == NULL, np == n).
 *   rows:     [np][W] membership of pids[k] (p in S_delta(P)).
 *   ext_rows: [np][W] or NULL, p in S+_delta(P). */
int oracle_b_rows(const float *pts, int64_t n, int d, const int64_t *pids, int64_t np,
                  uint32_t *rows, uint32_t *ext_rows) {
    if (d < 1 || d > 16 || n < 0) return 1;
    const uint32_t W = words_per_row(d);
    const uint32_t size = 1u << d;
    int status = 0;
    #pragma omp parallel
    {
        uint8_t *Gs = (uint8_t *)malloc(size);
        uint8_t *G = (uint8_t *)malloc((size_t)size * d);
        if (!Gs || !G) {
            #pragma omp atomic write
            status = 2;
        } else {
            #pragma omp for schedule(dynamic, 1)
            for (int64_t k = 0; k < np; k++) {
                const int64_t p = pids ? pids[k] : k;
                const float *pp = pts + (size_t)p * d;
                memset(Gs, 0, size);
                memset(G, 0, (size_t)size * d);
                for (int64_t q = 0; q < n; q++) {
                    if (q == p) continue;
                    uint32_t L, S;
                    relation_masks(pts + (size_t)q * d, pp, d, &L, &S);
                    if (!S) continue;                 /* no dimension where q is better */
                    Gs[S] = 1;
                    for (int i = 0; i < d; i++)
                        if (S & (1u << i)) G[(size_t)i * size + L] = 1;
                }
                superset_closure(Gs, d);
                for (int i = 0; i < d; i++) superset_closure(G + (size_t)i * size, d);
                uint32_t *row = rows + (size_t)k * W;
                uint32_t *erow = ext_rows ? ext_rows + (size_t)k * W : NULL;
                memset(row, 0, sizeof(uint32_t) * W);
                if (erow) memset(erow, 0, sizeof(uint32_t) * W);
                for (uint32_t delta = 1; delta < size; delta++) {
                    int dom = 0;
                    for (int i = 0; i < d && !dom; i++)
                        if ((delta & (1u << i)) && G[(size_t)i * size + delta]) dom = 1;
                    if (!dom) row[delta >> 5] |= 1u << (delta & 31);
                    if (erow && !Gs[delta]) erow[delta >> 5] |= 1u << (delta & 31);
                }
            }
        }
        free(Gs);
        free(G);
    }
    return status;
}

/* ---------------------------------------------------------------------------------------------
 * Lattice (Fig. 1a: "for each subspace delta, a flat array stores the point ids of S_delta")
 * from membership rows: offsets[2^d + 1], ids ascending within each delta (reading Q12).
 * Call once with ids == NULL to get offsets (total = offsets[2^d]), then again with ids.
 * ------------------------------------------------------------------------------------------- */
int oracle_lattice(const uint32_t *rows, int64_t n, int d, int64_t *offsets, int32_t *ids) {
    if (d < 1 || d > 16) return 1;
    const uint32_t W = words_per_row(d);
    const uint32_t size = 1u << d;
    memset(offsets, 0, sizeof(int64_t) * (size + 1));
    for (int64_t p = 0; p < n; p++)
        for (uint32_t delta = 1; delta < size; delta++)
            if (rows[(size_t)p * W + (delta >> 5)] & (1u << (delta & 31))) offsets[delta + 1]++;
    for (uint32_t delta = 0; delta < size; delta++) offsets[delta + 1] += offsets[delta];
    if (!ids) return 0;
    int64_t *cursor = (int64_t *)malloc(sizeof(int64_t) * size);
    if (!cursor) return 2;
    memcpy(cursor, offsets, sizeof(int64_t) * size);
    for (int64_t p = 0; p < n; p++)
        for (uint32_t delta = 1; delta < size; delta++)
            if (rows[(size_t)p * W + (delta >> 5)] & (1u << (delta & 31))) ids[cursor[delta]++] = (int32_t)p;
    free(cursor);
    return 0;
}
