/* sim_k3.c — CPU work model of K3 (design tool; not the oracle, not the product).
 *
 * Reproduces the GPU path's data layout on the host (order-preserving keys, 15-bit monotone codes, Morton
 * static-tree order, S+ by a K1-like scan, competitor chunks of 32 / sub-chunks of 4 with lower corners,
 * chunks visited by corner-code sum) and runs K3's per-task test cascade sequentially for a sample of
 * task groups (32 consecutive S+ points in a chosen task order), counting the tests each candidate design
 * executes.  The state is B_{p notin S+} (strict, downward closed) plus the tie part, exactly as the
 * kernel's kModeGlobalTie.  Skips are sound, so every variant below sees the same state trajectory; only
 * the number of tests differs:
 *   box        per (task, chunk): M = B_{corner<=p}; skip if M in state              (design A today)
 *   gbox       per (group, chunk): M_g = B_{corner<=U_g} (U_g = group's upper corner); a lane whose state
 *              holds M_g skips without its own mask; a warp-iteration is free iff all 32 lanes skip
 *   gtile      per (group, tile of 16 chunks): same with the tile's lower corner
 * Usage: sim_k3 points.f32 n d ngroups_sample task_order(0=id,1=morton) chunk_order(0=sum,1=morton,2=coarse)
 *        [chunk_size=32] [sub_size=4] [box_shift=0] [sub_shift=0] [prelude=0]
 */
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>
#include <omp.h>

static int D, N;
static uint32_t *ORD;     /* [N][D] order-preserving keys */
static uint16_t *CODE;    /* [N][D] codes */

static uint32_t ordkey(float x) {
    uint32_t b;
    memcpy(&b, &x, 4);
    if ((b & 0x7fffffffu) == 0) b = 0;
    return (b & 0x80000000u) ? ~b : (b | 0x80000000u);
}

static const uint32_t *g_sortkeys;
static int cmp_idx_u32(const void *a, const void *b) {
    uint32_t x = g_sortkeys[*(const int *)a], y = g_sortkeys[*(const int *)b];
    return x < y ? -1 : x > y;
}
static const uint64_t *g_sortkeys64;
static int cmp_idx_u64(const void *a, const void *b) {
    uint64_t x = g_sortkeys64[*(const int *)a], y = g_sortkeys64[*(const int *)b];
    if (x != y) return x < y ? -1 : 1;
    return *(const int *)a - *(const int *)b;
}

static inline uint32_t le_mask(const uint16_t *c, const uint16_t *p) { /* B_{c<=p} */
    uint32_t m = 0;
    for (int i = 0; i < D; i++) m |= (uint32_t)(c[i] <= p[i]) << i;
    return m;
}
static inline int bit(const uint32_t *st, uint32_t m) { return (st[m >> 5] >> (m & 31)) & 1u; }
static inline void set_sub(uint32_t *st, uint32_t S) { /* all non-empty subsets of S (and 0) */
    for (uint32_t s = S;; s = (s - 1) & S) {
        st[s >> 5] |= 1u << (s & 31);
        if (!s) break;
    }
}

int main(int argc, char **argv) {
    if (argc < 7) {
        fprintf(stderr, "usage\n");
        return 1;
    }
    N = atoi(argv[2]);
    D = atoi(argv[3]);
    const int nsample = atoi(argv[4]), task_order = atoi(argv[5]), chunk_order = atoi(argv[6]);
    const int CS = argc > 7 ? atoi(argv[7]) : 32, SS = argc > 8 ? atoi(argv[8]) : 4, NSUB = CS / SS;
    const int BOXSHIFT = argc > 9 ? atoi(argv[9]) : 0;  /* box test on codes >> BOXSHIFT (coarser, still sound) */
    const int SUBSHIFT = argc > 10 ? atoi(argv[10]) : 0;  /* sub-corner test on codes >> SUBSHIFT */
    /* prelude: before the global order, each group visits the PRE static-tree (Morton) chunks on either side of
     * its own position (meaningful with task_order = 1: group g = the members of chunk g) */
    const int PRE = argc > 11 ? atoi(argv[11]) : 0;
    float *X = malloc(sizeof(float) * N * D);
    FILE *f = fopen(argv[1], "rb");
    if (fread(X, sizeof(float), (size_t)N * D, f) != (size_t)N * D) return 2;
    fclose(f);
    ORD = malloc(sizeof(uint32_t) * N * D);
    CODE = malloc(sizeof(uint16_t) * N * D);
    for (long k = 0; k < (long)N * D; k++) ORD[k] = ordkey(X[k]);
    /* codes per dimension: dense rank, scaled to 15 bits when there are more than 2^15 distinct values */
    int *idx = malloc(sizeof(int) * N);
    uint32_t *col = malloc(sizeof(uint32_t) * N);
    uint32_t R[16];
    for (int i = 0; i < D; i++) {
        for (int p = 0; p < N; p++) idx[p] = p, col[p] = ORD[(long)p * D + i];
        g_sortkeys = col;
        qsort(idx, N, sizeof(int), cmp_idx_u32);
        uint32_t r = 0;
        for (int k = 0; k < N; k++) {
            if (k && col[idx[k]] != col[idx[k - 1]]) r++;
            col[idx[k]] = col[idx[k]];
            CODE[(long)idx[k] * D + i] = 0;
        }
        R[i] = r + 1;
        r = 0;
        uint32_t *rank = malloc(sizeof(uint32_t) * N);
        for (int k = 0; k < N; k++) {
            if (k && col[idx[k]] != col[idx[k - 1]]) r++;
            rank[idx[k]] = r;
        }
        for (int p = 0; p < N; p++)
            CODE[(long)p * D + i] = (uint16_t)(R[i] <= 32768 ? rank[p] : (uint32_t)(((uint64_t)rank[p] * 32768) / R[i]));
        free(rank);
    }
    /* Morton order of the (rescaled) codes */
    const int bpd = 64 / D < 15 ? 64 / D : 15;
    uint64_t *mk = malloc(sizeof(uint64_t) * N);
    for (int p = 0; p < N; p++) {
        uint64_t key = 0;
        for (int b = 0; b < bpd; b++)
            for (int i = 0; i < D; i++) {
                uint32_t c = CODE[(long)p * D + i];
                uint32_t sc = R[i] <= 32768 ? (uint32_t)(((uint64_t)c * 32768) / R[i]) : c;
                key = (key << 1) | ((sc >> (14 - b)) & 1u);
            }
        mk[p] = key;
    }
    int *mort = malloc(sizeof(int) * N);
    for (int p = 0; p < N; p++) mort[p] = p;
    g_sortkeys64 = mk;
    qsort(mort, N, sizeof(int), cmp_idx_u64);

    /* S+ : p in S+ iff no q with ORD[q] < ORD[p] in every dimension; candidates by key sum (Λ2) */
    uint64_t *ks = malloc(sizeof(uint64_t) * N);
    for (int p = 0; p < N; p++) {
        uint64_t s = 0;
        for (int i = 0; i < D; i++) s += ORD[(long)p * D + i];
        ks[p] = s;
    }
    int *byk = malloc(sizeof(int) * N);
    for (int p = 0; p < N; p++) byk[p] = p;
    g_sortkeys64 = ks;
    qsort(byk, N, sizeof(int), cmp_idx_u64);
    /* blocks of 32 in key order with lower corner (keys) for pruning */
    const int nb = (N + 31) / 32;
    uint32_t *bmin = malloc(sizeof(uint32_t) * nb * D);
    for (int b = 0; b < nb; b++)
        for (int i = 0; i < D; i++) {
            uint32_t m = 0xffffffffu;
            for (int k = b * 32; k < N && k < b * 32 + 32; k++) {
                uint32_t v = ORD[(long)byk[k] * D + i];
                if (v < m) m = v;
            }
            bmin[(long)b * D + i] = m;
        }
    uint8_t *ext = calloc(N, 1);
#pragma omp parallel for schedule(dynamic, 256)
    for (int k = 0; k < N; k++) {
        const int p = byk[k];
        const uint32_t *pp = ORD + (long)p * D;
        int dom = 0;
        for (int b = 0; b <= k / 32 && !dom; b++) {
            int ok = 1;
            for (int i = 0; i < D; i++) ok &= bmin[(long)b * D + i] < pp[i];
            if (!ok) continue;
            for (int t = b * 32; t < N && t < b * 32 + 32 && t < k && !dom; t++) {
                const uint32_t *qq = ORD + (long)byk[t] * D;
                int s = 1;
                for (int i = 0; i < D; i++) s &= qq[i] < pp[i];
                dom = s;
            }
        }
        ext[p] = !dom;
    }
    int m = 0;
    for (int p = 0; p < N; p++) m += ext[p];
    /* competitors: S+ in Morton order, chunks of 32 (padding never better) */
    int *qm = malloc(sizeof(int) * m);
    int mq = 0;
    for (int k = 0; k < N; k++)
        if (ext[mort[k]]) qm[mq++] = mort[k];
    const int nch = (m + CS - 1) / CS;
    uint16_t *corner = malloc(sizeof(uint16_t) * nch * D), *sub = malloc(sizeof(uint16_t) * nch * NSUB * D);
    for (int c = 0; c < nch; c++)
        for (int i = 0; i < D; i++) {
            uint16_t mn = 0x7fff;
            for (int s = 0; s < NSUB; s++) {
                uint16_t ms = 0x7fff;
                for (int r = 0; r < SS; r++) {
                    int k = c * CS + s * SS + r;
                    if (k < m && CODE[(long)qm[k] * D + i] < ms) ms = CODE[(long)qm[k] * D + i];
                }
                sub[((long)c * NSUB + s) * D + i] = ms;
                if (ms < mn) mn = ms;
            }
            corner[(long)c * D + i] = mn;
        }
    /* chunk visiting order */
    int *corder = malloc(sizeof(int) * nch);
    uint64_t *ck = malloc(sizeof(uint64_t) * nch);
    for (int c = 0; c < nch; c++) {
        uint64_t s = 0;
        for (int i = 0; i < D; i++) s += corner[(long)c * D + i];
        ck[c] = chunk_order == 0 ? s : chunk_order == 1 ? (uint64_t)c : (s >> 12) * (uint64_t)nch + c;
        corder[c] = c;
    }
    g_sortkeys64 = ck;
    qsort(corder, nch, sizeof(int), cmp_idx_u64);
    /* tile corners (16 consecutive visited chunks) */
    const int ntl = (nch + 15) / 16;
    uint16_t *tcorner = malloc(sizeof(uint16_t) * ntl * D);
    for (int t = 0; t < ntl; t++)
        for (int i = 0; i < D; i++) {
            uint16_t mn = 0x7fff;
            for (int k = t * 16; k < nch && k < t * 16 + 16; k++)
                if (corner[(long)corder[k] * D + i] < mn) mn = corner[(long)corder[k] * D + i];
            tcorner[(long)t * D + i] = mn;
        }
    /* tasks: S+ in id order (design A today) or Morton order; sample groups of 32 */
    int *tasks = malloc(sizeof(int) * m);
    if (task_order == 0) {
        int k = 0;
        for (int p = 0; p < N; p++)
            if (ext[p]) tasks[k++] = p;
    } else {
        memcpy(tasks, qm, sizeof(int) * m);
    }
    const int ngroups = m / 32;
    const int W = D >= 5 ? 1 << (D - 5) : 1;
    long long n_box = 0, n_sub = 0, n_pair = 0, n_miss = 0, n_exp = 0;
    long long g_lane_skip = 0, g_warp_free = 0, g_iters = 0, t_warp_free = 0, t_iters = 0;
    long long box_after_gtile = 0, n_half = 0, n_sub_h = 0, lb_sub = 0, lb_pair = 0, lb_open = 0;
#pragma omp parallel for schedule(dynamic, 1) reduction(+ : n_box, n_sub, n_pair, n_miss, n_exp, g_lane_skip, g_warp_free, g_iters, t_warp_free, t_iters, box_after_gtile, n_half, n_sub_h, lb_sub, lb_pair, lb_open)
    for (int sg = 0; sg < nsample; sg++) {
        const int g = (int)(((long long)sg * 7919 + 13) % ngroups);
        uint32_t *st = calloc((size_t)32 * W, 4), *tie = calloc((size_t)32 * W, 4);
        uint16_t U[16];
        for (int i = 0; i < D; i++) U[i] = 0;
        for (int l = 0; l < 32; l++) {
            st[l * W] = 1u;
            for (int i = 0; i < D; i++) {
                uint16_t c = CODE[(long)tasks[g * 32 + l] * D + i];
                if (c > U[i]) U[i] = c;
            }
        }
        for (int t = -1; t < ntl; t++) {
            int all = 0, k0, k1;
            if (t < 0) { /* prelude */
                k0 = -2 * PRE - 1;
                k1 = PRE > 0 ? 0 : k0;
            } else {
                /* tile-level group test */
                const uint32_t Mt = le_mask(tcorner + (long)t * D, U);
                all = 1;
                for (int l = 0; l < 32; l++) all &= bit(st + l * W, Mt);
                t_iters++;
                if (all) t_warp_free++;
                k0 = t * 16;
                k1 = k0 + 16 < nch ? k0 + 16 : nch;
            }
            for (int k = k0; k < k1; k++) {
                int c;
                if (k < 0) {
                    c = g + (k + PRE + 1);
                    if (c < 0 || c >= nch) continue;
                } else {
                    c = corder[k];
                }
                const uint16_t *cc = corner + (long)c * D;
                const uint32_t Mg = le_mask(cc, U);
                int allg = 1;
                for (int l = 0; l < 32; l++) {
                    uint32_t *sp = st + l * W, *tp = tie + l * W;
                    const int p = tasks[g * 32 + l];
                    const uint16_t *pc = CODE + (long)p * D;
                    const int gs = bit(sp, Mg);
                    g_lane_skip += gs;
                    allg &= gs;
                    n_box++;
                    if (!all) box_after_gtile++;
                    uint32_t Mb = 0;
                    for (int i = 0; i < D; i++) Mb |= (uint32_t)((cc[i] >> BOXSHIFT) <= (pc[i] >> BOXSHIFT)) << i;
                    if (bit(sp, Mb)) continue;
                    int half_open[2] = {1, 1};
                    if (NSUB == 8) {  /* three-level variant: half corners (16 points) before the sub-corners */
                        for (int h = 0; h < 2; h++) {
                            uint16_t hc[16];
                            for (int i = 0; i < D; i++) {
                                uint16_t mn = 0x7fff;
                                for (int s2 = 4 * h; s2 < 4 * h + 4; s2++)
                                    if (sub[((long)c * NSUB + s2) * D + i] < mn) mn = sub[((long)c * NSUB + s2) * D + i];
                                hc[i] = mn;
                            }
                            n_half++;
                            half_open[h] = !bit(sp, le_mask(hc, pc));
                            if (half_open[h]) n_sub_h += 4;
                        }
                    }
                    for (int s = 0; s < NSUB; s++) {
                        n_sub++;
                        {
                            const uint16_t *sc = sub + ((long)c * NSUB + s) * D;
                            uint32_t Ms = 0;
                            for (int i = 0; i < D; i++) Ms |= (uint32_t)((sc[i] >> SUBSHIFT) <= (pc[i] >> SUBSHIFT)) << i;
                            if (bit(sp, Ms)) continue;
                        }
                        for (int r = 0; r < SS; r++) {
                            const int kq = c * CS + s * SS + r;
                            if (kq >= m) continue;
                            n_pair++;
                            const int q = qm[kq];
                            const uint32_t M = le_mask(CODE + (long)q * D, pc);
                            if (bit(sp, M)) continue;
                            n_miss++;
                            uint32_t L = 0, S = 0;
                            for (int i = 0; i < D; i++) {
                                L |= (uint32_t)(ORD[(long)q * D + i] <= ORD[(long)p * D + i]) << i;
                                S |= (uint32_t)(ORD[(long)q * D + i] < ORD[(long)p * D + i]) << i;
                            }
                            if (!S || bit(sp, L)) continue;
                            n_exp++;
                            if (!bit(sp, S)) set_sub(sp, S);
                            if (L != S) { /* tie part: subsets of L that meet S */
                                for (uint32_t dd = L;; dd = (dd - 1) & L) {
                                    if (dd & S) tp[dd >> 5] |= 1u << (dd & 31);
                                    if (!dd) break;
                                }
                            }
                        }
                    }
                }
                g_iters++;
                g_warp_free += allg;
            }
        }
        /* lower bound for any visiting order: the tests a pass with the final (saturated) state still runs */
        for (int l = 0; l < 32; l++) {
            uint32_t *sp = st + l * W;
            const uint16_t *pc = CODE + (long)tasks[g * 32 + l] * D;
            for (int c = 0; c < nch; c++) {
                const uint16_t *cc = corner + (long)c * D;
                if (bit(sp, le_mask(cc, pc))) continue;
                lb_open++;
                for (int s2 = 0; s2 < NSUB; s2++) {
                    lb_sub++;
                    if (bit(sp, le_mask(sub + ((long)c * NSUB + s2) * D, pc))) continue;
                    lb_pair += SS;
                }
            }
        }
        free(st);
        free(tie);
    }
    const double scale = (double)ngroups / nsample;
    printf("{\"n\": %d, \"d\": %d, \"m\": %d, \"nchunks\": %d, \"chunk\": %d, \"sub\": %d, \"task_order\": %d, \"chunk_order\": %d, \"sample_groups\": %d,\n",
           N, D, m, nch, CS, SS, task_order, chunk_order, nsample);
    printf(" \"box\": %.4g, \"sub\": %.4g, \"pair\": %.4g, \"miss\": %.4g, \"expansions\": %.4g,\n", n_box * scale,
           n_sub * scale, n_pair * scale, n_miss * scale, n_exp * scale);
    printf(" \"three_level\": {\"half\": %.4g, \"sub\": %.4g},\n", n_half * scale, n_sub_h * scale);
    printf(" \"saturated_state_lower_bound\": {\"open\": %.4g, \"sub\": %.4g, \"pair\": %.4g},\n", lb_open * scale,
           lb_sub * scale, lb_pair * scale);
    printf(" \"gbox_lane_skip_frac\": %.4f, \"gbox_warp_free_frac\": %.4f, \"gtile_warp_free_frac\": %.4f,"
           " \"box_after_gtile_frac\": %.4f}\n",
           (double)g_lane_skip / n_box, (double)g_warp_free / g_iters, (double)t_warp_free / t_iters,
           (double)box_after_gtile / n_box);
    return 0;
}
