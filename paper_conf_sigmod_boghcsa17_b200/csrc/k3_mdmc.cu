// k3_mdmc.cu — K3: the MDMC per-point task of Alg. 3 (L313-319), lines 3-12, on sm_100a.
//
// For every p in S+(P) (the data-parallel tasks, L306-310) and every competitor q in S+(P) (Λ1:
// competitors outside S+ add nothing), the pair reduces to two d-bit masks (L77)
//     L = B_{q<=p},  S = B_{q<p}   (E = L \ S = B_{q=p})
// and q dominates p exactly in the subspaces { delta subset of L : delta & S != 0 } (Def. 1), strictly in the
// non-empty subsets of S.  B_{p notin S+} (strict) is downward closed, so bit L set in it means q adds
// nothing new (L330-336, Alg. 3 line 11) — the probe that skips almost every pair.
//
// Per pair, on the hot path:
//   1. M = B_{code(q)<=code(p)} by SWAR over 16-bit code lanes with a guard bit (2 dimensions per
//      32-bit subtraction), gathered to a d-bit mask with a byte permute and one multiply per 4
//      dimensions.  Codes are monotone (Λ3), so M is a superset of L (equal where codes are exact).
//   2. probe bit M of B_{p notin S+} in shared memory; set => skip (Λ4).
// Only on a miss (rare: < 1% of pairs):
//   3. S from the strict SWAR compare; exact refinement of the dimensions whose codes tie but are not
//      injective; then set sub(S) in B_{p notin S+} (Alg. 3 line 12, word-parallel), and, only when q
//      ties p somewhere (E != 0), the tie contribution sub(L) \ sub(E) in a global tie row (reading Q3).
//   B_{p notin S} = B_{p notin S+} | tie row; the membership row written out is its complement.
//
// Two layouts of the per-task state (the paper's thread-block-per-point of L498-512 is prior art):
//   design A (d <= 12): one thread per task p, a warp = 32 tasks, every competitor q is read once per
//     CTA from shared memory as a broadcast; B_{p notin S+} lives in shared memory as [word][lane]
//     (bank = lane, conflict-free probes).  2^d/8 bytes per task.
//   design B (d > 12): a CTA holds the states of NT tasks (192 KB in total, 8 KB per task at d = 16);
//     each lane holds one competitor in registers and runs it against all NT tasks (task codes are
//     broadcasts); misses expand with shared-memory atomics.
#include <algorithm>
#include <cstdlib>

#include "ctx.cuh"
#include "tile_stream.cuh"

namespace sky {
namespace {

template <int D>
struct Geo {
    static constexpr int DP = ((D + 3) / 4) * 4;
    static constexpr int CW = DP / 2;                       // 32-bit code words per point
    static constexpr int NG = DP / 4;                       // groups of 4 dimensions
    static constexpr int WB = D >= 5 ? (1 << (D - 5)) : 1;  // 32-bit words of a 2^d-bit state
    static constexpr uint32_t kRowMask = D >= 5 ? 0xffffffffu : ((1u << (1 << D)) - 1u);
};

// Mask of guard bits -> d-bit mask, dimension i -> bit i.  Word k holds dimensions 2k (bits 0-15) and
// 2k+1 (bits 16-31); guard bits at 15 and 31.  Per group of 4 dimensions: byte-permute the 4 guard
// bytes into one word, keep the MSBs, and move them to bits 28..31 with a carry-free multiply.
template <int NG>
__device__ __forceinline__ uint32_t gather_mask(const uint32_t *v) {
    uint32_t m = 0;
#pragma unroll
    for (int g = NG - 1; g >= 0; g--) {
        const uint32_t x = __byte_perm(v[2 * g], v[2 * g + 1], 0x7531) & 0x80808080u;
        const uint32_t y = x * 0x00204081u;  // byte k MSB (bit 8k+7) -> bit 28+k, no carries
        m = __funnelshift_l(y, m, 4);       // (m << 4) | (y >> 28)
    }
    return m;
}

// Bits delta_low (0..31) that are subsets of x (x < 32): the word pattern of sub(x) in the low 5 dims.
__device__ __forceinline__ uint32_t sub5(uint32_t x) {
    uint32_t t = 1u;
    if (x & 1u) t |= t << 1;
    if (x & 2u) t |= t << 2;
    if (x & 4u) t |= t << 4;
    if (x & 8u) t |= t << 8;
    if (x & 16u) t |= t << 16;
    return t;
}

// Exact refinement of the dimensions in U (codes tie, codes not injective there).
__device__ __forceinline__ void refine_exact(uint32_t U, const uint32_t *__restrict__ qo, const uint32_t *__restrict__ po,
                                             uint32_t &L, uint32_t &S) {
    while (U) {
        const int i = __ffs(U) - 1;
        U &= U - 1;
        const uint32_t qv = qo[i], pv = po[i];
        if (qv > pv) L &= ~(1u << i);
        else if (qv < pv) S |= 1u << i;
    }
}

// ==================================================================================== design A
constexpr int kAWarps = 4;
constexpr int kATQ = 128;  // competitors per shared-memory tile
constexpr int kAU = 8;     // competitors per inner iteration (independent chains for ILP)
constexpr int kAStages = 3;  // TMA ring depth

// The rare miss path for one (p, q) pair (Alg. 3 lines 10-12).  Returns true if a tie row was written.
// `tr` points at word 0 of the task's tie row, stride 32 words: shared memory (TIES layout) or global.
template <int D>
__device__ __forceinline__ bool mdmc_miss(uint32_t *st, const uint32_t *pH, const uint32_t *qw, uint32_t M,
                                          uint32_t inexact, const uint32_t *__restrict__ qo,
                                          const uint32_t *__restrict__ po, uint32_t *tr) {
    using G = Geo<D>;
    uint32_t lt[G::CW];
#pragma unroll
    for (int k = 0; k < G::CW; k++) lt[k] = pH[k] - qw[k] - 0x00010001u;  // guard <=> code(q) < code(p)
    uint32_t S = gather_mask<G::NG>(lt);
    uint32_t L = M;
    const uint32_t U = M & ~S & inexact;
    if (U) refine_exact(U, qo, po, L, S);
    if (S == 0) return false;                                         // q is nowhere better than p
    if (L != M && ((st[(L >> 5) * 32] >> (L & 31)) & 1u)) return false;
    if (!((st[(S >> 5) * 32] >> (S & 31)) & 1u)) {  // B_{p notin S+} |= sub(S) (strict dominance propagates)
        const uint32_t sh = S >> 5, bits = sub5(S & 31u);
        uint32_t w = 0;
        do {
            st[w * 32] |= bits;
            w = (w - sh) & sh;
        } while (w);
    }
    if (L == S) return false;
    // ties: B_{p notin S} |= sub(L) \ sub(E), E = B_{q=p}  (reading Q3)
    const uint32_t E = L & ~S;
    const uint32_t lh = L >> 5, eh = E >> 5, lb = sub5(L & 31u), eb = sub5(E & 31u);
    uint32_t w = 0;
    do {
        tr[w * 32] |= (w & ~eh) ? lb : (lb & ~eb);
        w = (w - lh) & lh;
    } while (w);
    return true;
}

template <int D, bool TIES>
__global__ void __launch_bounds__((kAWarps + 1) * 32) k3_mdmc_a_kernel(
    const uint32_t *__restrict__ p_codes, const uint32_t *__restrict__ p_ord, const uint32_t *__restrict__ q_codes,
    const uint32_t *__restrict__ q_ord, int64_t ntiles_q, int64_t j_begin, int64_t j_end, uint32_t inexact,
    uint32_t *__restrict__ rows32, uint32_t *__restrict__ tie32, uint32_t *__restrict__ ext_rows32) {
    using G = Geo<D>;
    extern __shared__ __align__(128) uint32_t smem[];
    uint64_t *bars = reinterpret_cast<uint64_t *>(smem);             // full[kAStages], empty[kAStages]
    const TileRing<kAStages> ring{bars, bars + kAStages, smem + 4 * kAStages, (uint32_t)(kATQ * G::CW)};
    uint32_t *stbase = smem + 4 * kAStages + kAStages * kATQ * G::CW;  // [kAWarps][WB][32]
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    uint32_t *st = stbase + warp * G::WB * 32 + lane;                // word w of this task: st[w * 32]
    const int64_t j = j_begin + (int64_t)blockIdx.x * (kAWarps * 32) + warp * 32 + lane;
    const bool active = j < j_end;
    const int64_t grp = j >> 5;
    // TIES: the tie part of B_{p notin S} also lives in shared memory (tie-heavy / low-d inputs)
    uint32_t *tr = TIES ? stbase + (kAWarps + warp) * G::WB * 32 + lane : tie32 + grp * (G::WB * 32) + lane;

    if (threadIdx.x == 0) ring.init(kAWarps);
    if (warp == kAWarps) {  // producer warp: one elected lane streams competitor tiles with TMA
        __syncthreads();
        if (lane == 0)
            for (int64_t t = 0; t < ntiles_q; t++) ring.issue(q_codes, t);
        return;
    }
    uint32_t pH[G::CW];
#pragma unroll
    for (int k = 0; k < G::CW; k++) {
        uint32_t w = active ? p_codes[j * G::CW + k] : 0u;
        if (2 * k >= D) w &= 0xffff0000u;  // padding dimensions: p = 0 never passes q <= p (q pad = 1)
        if (2 * k + 1 >= D) w &= 0x0000ffffu;
        pH[k] = w | kGuard;
    }
#pragma unroll 4
    for (int w = 0; w < G::WB; w++) {
        st[w * 32] = w == 0 ? 1u : 0u;  // bit 0 (empty subspace) preset
        if (TIES) tr[w * 32] = 0u;
    }
    bool had_tie = false;
    __syncthreads();
    const char *stc = reinterpret_cast<const char *>(st);

    for (int64_t tq = 0; tq < ntiles_q; tq++) {
        ring.wait(tq);
        const uint32_t *qs = ring.stage(tq);
        if (active) {
#pragma unroll 1
            for (int t = 0; t < kATQ; t += kAU) {
                uint32_t M[kAU], wd[kAU];
#pragma unroll
                for (int u = 0; u < kAU; u++) {
                    const uint32_t *qw = qs + (t + u) * G::CW;
                    uint32_t le[G::CW];
#pragma unroll
                    for (int k = 0; k < G::CW; k++) le[k] = pH[k] - qw[k];  // guard <=> code(q) <= code(p)
                    M[u] = gather_mask<G::NG>(le);
                }
#pragma unroll
                for (int u = 0; u < kAU; u++) wd[u] = *reinterpret_cast<const uint32_t *>(stc + ((M[u] >> 5) << 7));
                uint32_t hit = 0xffffffffu;
#pragma unroll
                for (int u = 0; u < kAU; u++) hit &= __funnelshift_r(wd[u], wd[u], M[u]);  // bit M of B_{p notin S+}
                if (hit & 1u) continue;                                   // Λ4: none of the kAU competitors adds anything
#pragma unroll
                for (int u = 0; u < kAU; u++) {
                    if ((st[(M[u] >> 5) * 32] >> (M[u] & 31)) & 1u) continue;
                    const int64_t q = tq * kATQ + t + u;
                    had_tie |= mdmc_miss<D>(st, pH, qs + (t + u) * G::CW, M[u], inexact, q_ord + q * D, p_ord + j * D, tr);
                }
            }
        }
        __syncwarp();
        if (lane == 0) ring.release(tq);
    }
    if (!active) return;
    uint32_t *out = rows32 + grp * (G::WB * 32) + lane;
#pragma unroll 4
    for (int w = 0; w < G::WB; w++) {
        uint32_t v = st[w * 32];
        if (TIES || had_tie) v |= tr[w * 32];
        uint32_t row = ~v & G::kRowMask;
        if (w == 0) row &= ~1u;
        out[w * 32] = row;
        if (ext_rows32) {
            uint32_t er = ~st[w * 32] & G::kRowMask;
            if (w == 0) er &= ~1u;
            ext_rows32[grp * (G::WB * 32) + w * 32 + lane] = er;
        }
    }
}

// ==================================================================================== design B
// d > 12: the 2^d-bit state (1-8 KB per task) is too large for one task per thread.  A CTA keeps the
// states of NT tasks in shared memory and every consumer warp holds 32 competitors in registers (one
// per lane, read once from the TMA-fed tile) and runs them against all NT tasks: the task's codes are
// a shared-memory broadcast, the probe goes to the task's state (random words: some bank conflicts),
// misses expand with shared-memory atomics (several warps may update one task's state).
constexpr int kBWarps = 16;           // consumer warps (+1 producer warp)
constexpr int kBTQ = kBWarps * 32;    // competitors per tile: one per consumer lane
constexpr int kBStages = 3;
constexpr int kBStateBytes = 160 * 1024;
constexpr int kBTU = 4;               // tasks per inner iteration (independent chains)

template <int D>
struct GeoB {
    static constexpr int NT = kBStateBytes / (Geo<D>::WB * 4) < 256 ? kBStateBytes / (Geo<D>::WB * 4) : 256;
};

template <int D>
__device__ __forceinline__ void mdmc_miss_b(uint32_t *st, const uint32_t *pH, const uint32_t *qw, uint32_t M,
                                            uint32_t inexact, const uint32_t *__restrict__ qo,
                                            const uint32_t *__restrict__ po, uint32_t *tr) {
    using G = Geo<D>;
    uint32_t lt[G::CW];
#pragma unroll
    for (int k = 0; k < G::CW; k++) lt[k] = pH[k] - qw[k] - 0x00010001u;
    uint32_t S = gather_mask<G::NG>(lt);
    uint32_t L = M;
    const uint32_t U = M & ~S & inexact;
    if (U) refine_exact(U, qo, po, L, S);
    if (S == 0) return;
    if (L != M && ((st[L >> 5] >> (L & 31)) & 1u)) return;
    if (!((st[S >> 5] >> (S & 31)) & 1u)) {
        const uint32_t sh = S >> 5, bits = sub5(S & 31u);
        uint32_t w = 0;
        do {
            atomicOr(&st[w], bits);
            w = (w - sh) & sh;
        } while (w);
    }
    if (L == S) return;
    const uint32_t E = L & ~S;
    const uint32_t lh = L >> 5, eh = E >> 5, lb = sub5(L & 31u), eb = sub5(E & 31u);
    uint32_t w = 0;
    do {
        atomicOr(&tr[w * 32], (w & ~eh) ? lb : (lb & ~eb));
        w = (w - lh) & lh;
    } while (w);
}

template <int D>
__global__ void __launch_bounds__((kBWarps + 1) * 32, 1) k3_mdmc_b_kernel(
    const uint32_t *__restrict__ p_codes, const uint32_t *__restrict__ p_ord, const uint32_t *__restrict__ q_codes,
    const uint32_t *__restrict__ q_ord, int64_t ntiles_q, int64_t j_begin, int64_t j_end, uint32_t inexact,
    uint32_t *__restrict__ rows32, uint32_t *__restrict__ tie32, uint32_t *__restrict__ ext_rows32) {
    using G = Geo<D>;
    constexpr int NT = GeoB<D>::NT;
    extern __shared__ __align__(128) uint32_t smem[];
    uint64_t *bars = reinterpret_cast<uint64_t *>(smem);
    const TileRing<kBStages> ring{bars, bars + kBStages, smem + 4 * kBStages, (uint32_t)(kBTQ * G::CW)};
    uint32_t *pcs = smem + 4 * kBStages + kBStages * kBTQ * G::CW;  // [NT][CW] task codes (with guard bits)
    uint32_t *state = pcs + NT * G::CW;                              // [NT][WB]
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int64_t j0 = j_begin + (int64_t)blockIdx.x * NT;
    const int nt = (int)min((int64_t)NT, j_end - j0);

    if (threadIdx.x == 0) ring.init(kBWarps);
    for (int i = threadIdx.x; i < NT * G::CW; i += blockDim.x) {
        const int t = i / G::CW, k = i % G::CW;
        uint32_t w = t < nt ? p_codes[(j0 + t) * G::CW + k] : 0u;
        if (2 * k >= D) w &= 0xffff0000u;
        if (2 * k + 1 >= D) w &= 0x0000ffffu;
        pcs[i] = w | kGuard;
    }
    for (int i = threadIdx.x; i < NT * G::WB; i += blockDim.x) state[i] = (i % G::WB) == 0 ? 1u : 0u;
    __syncthreads();
    if (warp == kBWarps) {  // producer warp
        if (lane == 0)
            for (int64_t t = 0; t < ntiles_q; t++) ring.issue(q_codes, t);
        return;
    }
    for (int64_t tq = 0; tq < ntiles_q; tq++) {
        ring.wait(tq);
        uint32_t qw[G::CW];
        const uint32_t *qsrc = ring.stage(tq) + (warp * 32 + lane) * G::CW;
#pragma unroll
        for (int k = 0; k < G::CW; k++) qw[k] = qsrc[k];
        __syncwarp();
        if (lane == 0) ring.release(tq);
        const int64_t q = tq * kBTQ + warp * 32 + lane;
#pragma unroll 1
        for (int t0 = 0; t0 < nt; t0 += kBTU) {
            uint32_t M[kBTU], wd[kBTU];
#pragma unroll
            for (int u = 0; u < kBTU; u++) {
                const int t = min(t0 + u, nt - 1);
                const uint32_t *ph = pcs + t * G::CW;
                uint32_t le[G::CW];
#pragma unroll
                for (int k = 0; k < G::CW; k++) le[k] = ph[k] - qw[k];
                M[u] = gather_mask<G::NG>(le);
                wd[u] = state[t * G::WB + (M[u] >> 5)];
            }
            uint32_t hit = 0xffffffffu;
#pragma unroll
            for (int u = 0; u < kBTU; u++) hit &= __funnelshift_r(wd[u], wd[u], M[u]);
            if (hit & 1u) continue;
#pragma unroll
            for (int u = 0; u < kBTU; u++) {
                const int t = t0 + u;
                if (t >= nt) break;
                uint32_t *st = state + t * G::WB;
                if ((st[M[u] >> 5] >> (M[u] & 31)) & 1u) continue;
                const int64_t jt = j0 + t;
                mdmc_miss_b<D>(st, pcs + t * G::CW, qw, M[u], inexact, q_ord + q * D, p_ord + jt * D,
                               tie32 + (jt >> 5) * (G::WB * 32) + (jt & 31));
            }
        }
    }
    // consumer warps only (the producer has returned): named barrier 1
    asm volatile("bar.sync 1, %0;" ::"r"(kBWarps * 32) : "memory");
    for (int t = warp; t < nt; t += kBWarps) {
        const int64_t jt = j0 + t;
        const uint32_t *st = state + t * G::WB;
        uint32_t *out = rows32 + (jt >> 5) * (G::WB * 32) + (jt & 31);
        const uint32_t *tr = tie32 + (jt >> 5) * (G::WB * 32) + (jt & 31);
        for (int w = lane; w < G::WB; w += 32) {
            const uint32_t v = st[w] | tr[w * 32];
            uint32_t row = ~v;
            if (w == 0) row &= ~1u;
            out[w * 32] = row;
            if (ext_rows32) {
                uint32_t er = ~st[w];
                if (w == 0) er &= ~1u;
                ext_rows32[(jt >> 5) * (G::WB * 32) + w * 32 + (jt & 31)] = er;
            }
        }
    }
}

// ==================================================================================== design C
// Static-tree chunk pruning (any d).  Competitors are S+ in static-tree (Morton) order, in chunks of 32
// with their lower corner.  For a task p and a chunk, Mbox = B_{corner<=p} is a superset of M(q,p) for
// every q of the chunk, so bit Mbox set in B_{p notin S+} proves the whole chunk adds nothing (Λ4 on a
// leaf range: the paper's filter on path labels, L320-328, with the tree's global pivots).  A CTA holds
// NT tasks; each consumer warp takes one chunk per tile (one competitor per lane, in registers):
//   box pass   lane l tests task g*32+l against the chunk corner; a ballot gives the tasks to refine;
//   pair pass  for each such task (4 at a time) every lane tests its competitor (task codes are a
//              shared-memory broadcast) and probes the task's state; misses run Alg. 3 lines 10-12 with
//              shared-memory atomics (several warps may update one task).
constexpr int kCWarps = 16;
constexpr int kCStages = 4;
constexpr int kCSmemBytes = 227 * 1024;  // opt-in maximum per CTA
constexpr int kCU = 4;

// CW words from a 16-byte aligned row (CW even): LDS.128 / LDS.64 instead of CW scalar loads.
template <int CW>
__device__ __forceinline__ void load_row(const uint32_t *p, uint32_t *w) {
#pragma unroll
    for (int k = 0; k + 4 <= CW; k += 4) {
        const uint4 v = *reinterpret_cast<const uint4 *>(p + k);
        w[k] = v.x;
        w[k + 1] = v.y;
        w[k + 2] = v.z;
        w[k + 3] = v.w;
    }
    if (CW % 4) {
        const uint2 v = *reinterpret_cast<const uint2 *>(p + (CW & ~3));
        w[CW & ~3] = v.x;
        w[(CW & ~3) + 1] = v.y;
    }
}

// State modes of design C (per task, in shared memory):
//   kModeGlobalTie  B_{p notin S+} (the probe set); the tie part of B_{p notin S} in a global row (continuous data)
//   kModeSmemTie    B_{p notin S+} and the tie part, both in shared memory
//   kModeDims       tie-exact state (reading Q3/Q4 made cheap under heavy ties): one downward-closed set per
//                   dimension, D_i = union of sub(L_q) over the q with i in S_q, and the probe set
//                   K = { delta : delta in D_i for every i in delta \ Z_p } (Z_p: dimensions where p holds the
//                   global minimum, so no q is strictly better there).  p is dominated in delta <=> delta in D_i
//                   for some i in delta (Def. 1: delta subset of L_q and delta & S_q != 0), and bit M in K proves
//                   that q (S_q subset of L_q \ Z_p, L_q subset of M) adds nothing to any D_i.  Without ties K is
//                   B_{p notin S+}; with ties K keeps growing where B_{p notin S+} cannot (ties at the optimum).
constexpr int kModeGlobalTie = 0, kModeSmemTie = 1, kModeDims = 2;

template <int D, int MODE>
struct GeoC {
    static constexpr int PER = (MODE == kModeGlobalTie ? 1 : MODE == kModeSmemTie ? 2 : D + 1) * Geo<D>::WB;
    static constexpr int PS = PER | 1;  // odd task stride: equal word indices of 32 tasks hit 32 banks
    static constexpr int ROW = PS + ((Geo<D>::CW + 3) & ~3) + (Geo<D>::CW | 1);  // words per task
    static constexpr int TW = kCWarps * 33 * Geo<D>::CW + ((Geo<D>::CW + 3) & ~3);  // tile: 16 chunks + super corner
    static constexpr int RING = 4 * kCStages + kCStages * TW;  // words
    static constexpr int NT0 = (kCSmemBytes / 4 - RING - 128 - kCWarps * 128) / (ROW + 1 + 1);
    static constexpr int NT = NT0 < 1024 ? NT0 : 1024;                         // tasks per CTA
};

template <int D>
__device__ __forceinline__ void mdmc_miss_c(uint32_t *st, const uint32_t *ph, const uint32_t *q, uint32_t M,
                                            uint32_t inexact, const uint32_t *__restrict__ qo,
                                            const uint32_t *__restrict__ po, uint32_t *tr, int tstride) {
    using G = Geo<D>;
    uint32_t lt[G::CW];
#pragma unroll
    for (int k = 0; k < G::CW; k++) lt[k] = ph[k] - q[k] - 0x00010001u;
    uint32_t S = gather_mask<G::NG>(lt);
    uint32_t L = M;
    const uint32_t U = M & ~S & inexact;
    if (U) refine_exact(U, qo, po, L, S);
    if (S == 0) return;
    if (L != M && ((st[L >> 5] >> (L & 31)) & 1u)) return;
    if (!((st[S >> 5] >> (S & 31)) & 1u)) {
        const uint32_t sh = S >> 5, bits = sub5(S & 31u);
        uint32_t w = 0;
        do {
            atomicOr(&st[w], bits);
            w = (w - sh) & sh;
        } while (w);
    }
    if (L == S) return;
    const uint32_t E = L & ~S;
    const uint32_t lh = L >> 5, eh = E >> 5, lb = sub5(L & 31u), eb = sub5(E & 31u);
    uint32_t w = 0;
    do {
        atomicOr(&tr[w * tstride], (w & ~eh) ? lb : (lb & ~eb));
        w = (w - lh) & lh;
    } while (w);
}

// Exact B_{q<=p}, B_{q<p} from the guard-bit compares plus exact keys on tied, non-injective codes.
template <int D>
__device__ __forceinline__ void exact_masks(const uint32_t *ph, const uint32_t *q, uint32_t M, uint32_t inexact,
                                            const uint32_t *__restrict__ qo, const uint32_t *__restrict__ po,
                                            uint32_t &L, uint32_t &S);

// Word pattern of the low-5-bit subspaces that contain dimension i (i < 5).
__device__ __forceinline__ uint32_t low_dim_pattern(int i) {
    return i == 0 ? 0xaaaaaaaau : i == 1 ? 0xccccccccu : i == 2 ? 0xf0f0f0f0u : i == 3 ? 0xff00ff00u : 0xffff0000u;
}

// kModeDims miss path (Alg. 3 lines 10-12 on the per-dimension sets).  st = [K | D_0 | ... | D_{d-1}].
template <int D>
__device__ __forceinline__ void mdmc_miss_dims(uint32_t *st, const uint32_t *ph, const uint32_t *q, uint32_t M,
                                               uint32_t inexact, const uint32_t *__restrict__ qo,
                                               const uint32_t *__restrict__ po, uint32_t z) {
    using G = Geo<D>;
    uint32_t L, S;
    exact_masks<D>(ph, q, M, inexact, qo, po, L, S);
    if (S == 0) return;                                              // q is nowhere better than p
    if (L != M && ((st[L >> 5] >> (L & 31)) & 1u)) return;           // exact L already covered by K
    const uint32_t lh = L >> 5, lb = sub5(L & 31u);
    bool changed = false;
    for (uint32_t s = S; s; s &= s - 1) {                            // D_i |= sub(L) for every i in S
        uint32_t *Di = st + (1 + (__ffs(s) - 1)) * G::WB;
        if ((Di[lh] >> (L & 31)) & 1u) continue;                     // downward closed: sub(L) already there
        changed = true;
        uint32_t w = 0;
        do {
            atomicOr(&Di[w], lb);
            w = (w - lh) & lh;
        } while (w);
    }
    if (!changed) return;
    // K on the words of sub(L) (only there can D change).  Racing warps may compute K from stale D words:
    // that only leaves K smaller (still sound); bits are only ever OR-ed in.
    const volatile uint32_t *vs = st;
    uint32_t w = 0;
    do {
        uint32_t k = 0xffffffffu;
#pragma unroll
        for (int i = 0; i < D; i++) {
            if ((z >> i) & 1u) continue;
            const uint32_t in = i < 5 ? low_dim_pattern(i) : (((w >> (i - 5)) & 1u) ? 0xffffffffu : 0u);
            k &= vs[(1 + i) * G::WB + w] | ~in;
        }
        atomicOr(&st[w], k);
        w = (w - lh) & lh;
    } while (w);
}

// Exact B_{q<=p}, B_{q<p} from the guard-bit compares plus exact keys on tied, non-injective codes.
template <int D>
__device__ __forceinline__ void exact_masks(const uint32_t *ph, const uint32_t *q, uint32_t M, uint32_t inexact,
                                            const uint32_t *__restrict__ qo, const uint32_t *__restrict__ po,
                                            uint32_t &L, uint32_t &S) {
    using G = Geo<D>;
    uint32_t lt[G::CW];
#pragma unroll
    for (int k = 0; k < G::CW; k++) lt[k] = ph[k] - q[k] - 0x00010001u;
    S = gather_mask<G::NG>(lt);
    L = M;
    const uint32_t U = M & ~S & inexact;
    if (U) refine_exact(U, qo, po, L, S);
}

// Warp-cooperative word-parallel expansion: dst |= { delta subset of X : not delta subset of E } (E subset X);
// E = 0 gives sub(X) (the empty set included, harmless: bit 0 is cleared on output).  Word w of dst at
// dst[w * stride].  The lanes take the subsets of the lowest five word-index bits of X; every lane
// iterates the subsets of the remaining word-index bits.  Atomic: other warps update the same task.
__device__ __forceinline__ void coop_down_or(uint32_t *dst, int stride, uint32_t X, uint32_t E, int lane) {
    const uint32_t xh = X >> 5, eh = E >> 5;
    const uint32_t xb = sub5(X & 31u), eb = sub5(E & 31u);
    uint32_t rest = xh, w_lo = 0;
    int np = 0;
#pragma unroll
    for (int i = 0; i < 5; i++) {
        if (rest) {
            const uint32_t bit = rest & (0u - rest);
            rest &= rest - 1;
            if ((lane >> i) & 1) w_lo |= bit;
            np++;
        }
    }
    if (lane < (1 << np)) {
        uint32_t w_hi = 0;
        do {
            const uint32_t w = w_lo | w_hi;
            const uint32_t bits = (w & ~eh) ? xb : (xb & ~eb);
            if (bits) atomicOr(&dst[w * stride], bits);
            w_hi = (w_hi - rest) & rest;
        } while (w_hi);
    }
    __syncwarp();
}

template <int D, int MODE>
__global__ void __launch_bounds__((kCWarps + 1) * 32, 1) k3_mdmc_c_kernel(
    const uint32_t *__restrict__ p_codes, const uint32_t *__restrict__ p_ord, const uint32_t *__restrict__ chunks,
    const uint32_t *__restrict__ q_ord, const uint32_t *__restrict__ minord, const uint32_t *__restrict__ supers,
    int use_super, int64_t nchunks, int64_t j_begin, int64_t j_end, uint32_t inexact, int tpc,
    uint32_t *__restrict__ rows32, uint32_t *__restrict__ tie32, uint32_t *__restrict__ ext_rows32,
    unsigned long long *__restrict__ counters) {
    using G = Geo<D>;
    using C = GeoC<D, MODE>;
    constexpr bool TIES = MODE == kModeSmemTie;
    constexpr int CWP = G::CW | 1;           // odd stride: per-lane row loads are conflict-free (box pass)
    constexpr int CWV = (G::CW + 3) & ~3;    // 16-byte stride: broadcast vector loads (pair pass)
    constexpr int REC = 33 * G::CW;
    extern __shared__ __align__(128) uint32_t smem[];
    uint64_t *bars = reinterpret_cast<uint64_t *>(smem);
    const TileRing<kCStages> ring{bars, bars + kCStages, smem + 4 * kCStages, (uint32_t)C::TW};
    uint32_t *pV = smem + 4 * kCStages + kCStages * C::TW;          // [tpc][CWV]
    uint32_t *pH = pV + tpc * CWV;                                   // [tpc][CWP]
    uint32_t *state = pH + tpc * CWP;                                // [tpc][PER]
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    uint32_t *zm = state + tpc * C::PS;                             // [tpc] Z_p (kModeDims)
    const int TG = (tpc + 31) >> 5;
    uint32_t *needw = zm + tpc;                                      // [2][TG] tasks below the tile corner
    uint32_t *mq = needw + 2 * TG + warp * 128;                      // per-warp miss queue [32][2]
    uint32_t *wq = mq + 64;                                          // per-warp pair-test task queue [36]
    const int64_t j0 = j_begin + (int64_t)blockIdx.x * tpc;
    const int nt = (int)min((int64_t)tpc, j_end - j0);
    const int64_t ntiles = ceil_div_dev(nchunks, kCWarps);

    if (threadIdx.x == 0) ring.init(kCWarps);
    for (int i = threadIdx.x; i < tpc * G::CW; i += blockDim.x) {
        const int t = i / G::CW, k = i % G::CW;
        uint32_t w = t < nt ? p_codes[(j0 + t) * G::CW + k] : 0u;
        if (2 * k >= D) w &= 0xffff0000u;  // padding dimensions: p = 0 never passes q <= p (q pad = 1)
        if (2 * k + 1 >= D) w &= 0x0000ffffu;
        pH[t * CWP + k] = w | kGuard;
        pV[t * CWV + k] = w | kGuard;
    }
    if (MODE == kModeDims) {
        // Z_p = { i : p[i] is the minimum of dimension i } (exact keys); K starts as sub(Z_p)
        for (int t = threadIdx.x; t < tpc; t += blockDim.x) {
            uint32_t z = 0;
            if (t < nt)
                for (int i = 0; i < D; i++)
                    if (p_ord[(j0 + t) * D + i] == minord[i]) z |= 1u << i;
            zm[t] = z;
        }
        __syncthreads();
        for (int i = threadIdx.x; i < tpc * C::PS; i += blockDim.x) {
            const int t = i / C::PS, w = i % C::PS;
            const uint32_t z = zm[t], zh = z >> 5;
            state[i] = w < G::WB && (w & ~zh) == 0 ? sub5(z & 31u) : 0u;
        }
    } else {
        for (int i = threadIdx.x; i < tpc * C::PS; i += blockDim.x) state[i] = (i % C::PS) == 0 ? 1u : 0u;
    }
    __syncthreads();
    if (warp == kCWarps) {
        if (lane == 0)
            for (int64_t t = 0; t < ntiles; t++) ring.issue2(chunks, kCWarps * REC, supers, (G::CW + 3) & ~3, t);
        return;
    }
    const int ngroups = (nt + 31) >> 5;
    unsigned long long n_box = 0, n_pair = 0, n_miss = 0;
    for (int64_t tile = 0; tile < ntiles; tile++) {
        ring.wait(tile);
        uint32_t *need = needw + (tile & 1) * TG;
        if (use_super) {
            // phase A (upper level of the static tree): tasks whose B_{p notin S+} (or K) already holds the mask
            // of the tile's lower corner skip all 16 chunks of the tile (Λ4 on 512 competitors at once)
            uint32_t sc[G::CW];
#pragma unroll
            for (int k = 0; k < G::CW; k++) sc[k] = ring.stage(tile)[kCWarps * REC + k];
            for (int g = warp; g < ngroups; g += kCWarps) {
                const int tt = min(g * 32 + lane, nt - 1);
                uint32_t le[G::CW];
#pragma unroll
                for (int k = 0; k < G::CW; k++) le[k] = pH[tt * CWP + k] - sc[k];
                const uint32_t Ms = gather_mask<G::NG>(le);
                const uint32_t ws = state[tt * C::PS + (Ms >> 5)];
                const uint32_t nb = __ballot_sync(0xffffffffu, g * 32 + lane < nt && !(__funnelshift_r(ws, ws, Ms) & 1u));
                if (lane == 0) need[g] = nb;
                n_box += min(32, nt - g * 32);
            }
            consumer_sync(kCWarps * 32);
        }
        const uint32_t *rec = ring.stage(tile) + warp * REC;
        uint32_t q[G::CW], mn[G::CW];
#pragma unroll
        for (int k = 0; k < G::CW; k++) {
            q[k] = rec[lane * G::CW + k];
            mn[k] = rec[32 * G::CW + k];
        }
        __syncwarp();
        if (lane == 0) ring.release(tile);
        const int64_t c = tile * kCWarps + warp;
        if (c >= nchunks) continue;
        const int64_t qpos = c * 32 + lane;
        // Pair tests are pooled across task groups in a per-warp queue and run kCU tasks at a time (independent
        // chains), so that a batch is only partial once per chunk.
        auto run_batch = [&](const int *ts, int cnt) {
                uint32_t M[kCU], wd[kCU];
#pragma unroll
                for (int u = 0; u < kCU; u++) {
                    uint32_t x[G::CW];
                    load_row<G::CW>(pV + ts[u] * CWV, x);
#pragma unroll
                    for (int k = 0; k < G::CW; k++) x[k] -= q[k];
                    M[u] = gather_mask<G::NG>(x);
                    wd[u] = state[ts[u] * C::PS + (M[u] >> 5)];
                }
                uint32_t hit = 0xffffffffu;
#pragma unroll
                for (int u = 0; u < kCU; u++) hit &= __funnelshift_r(wd[u], wd[u], M[u]);
                if (hit & 1u) return;
#pragma unroll
                for (int u = 0; u < kCU; u++) {
                    if (u >= cnt) break;
                    uint32_t *st = state + ts[u] * C::PS;
                    const int64_t jt = j0 + ts[u];
#ifndef SKY_COOP_MISS
                    if ((st[M[u] >> 5] >> (M[u] & 31)) & 1u) continue;
                    n_miss++;
                    if (MODE == kModeDims) {
                        mdmc_miss_dims<D>(st, pH + ts[u] * CWP, q, M[u], inexact, q_ord + qpos * D, p_ord + jt * D,
                                          zm[ts[u]]);
                    } else {
                        uint32_t *tr = TIES ? st + G::WB : tie32 + (jt >> 5) * (G::WB * 32) + (jt & 31);
                        mdmc_miss_c<D>(st, pH + ts[u] * CWP, q, M[u], inexact, q_ord + qpos * D, p_ord + jt * D, tr,
                                       TIES ? 1 : 32);
                    }
#else
                    // lane-local exact masks for the lanes that missed (Alg. 3 lines 10-11)
                    uint32_t L = 0, S = 0;
                    if (!((st[M[u] >> 5] >> (M[u] & 31)) & 1u)) {
                        n_miss++;
                        exact_masks<D>(pH + ts[u] * CWP, q, M[u], inexact, q_ord + qpos * D, p_ord + jt * D, L, S);
                        if (L != M[u] && ((st[L >> 5] >> (L & 31)) & 1u)) S = 0;
                    }
                    // line 12, warp-cooperative: contributing competitors are queued in shared memory (explicit
                    // reconvergence, no shuffles in divergent code), then all lanes expand each one
                    const uint32_t todo_m = __ballot_sync(0xffffffffu, S != 0);
                    if (S != 0) {
                        const int slot = __popc(todo_m & ((1u << lane) - 1u));
                        mq[2 * slot] = S;
                        mq[2 * slot + 1] = L;
                    }
                    __syncwarp();
                    const int nq = __popc(todo_m);
                    for (int e = 0; e < nq; e++) {
                        const uint32_t Sb = mq[2 * e], Lb = mq[2 * e + 1];
                        const uint32_t sw = st[Sb >> 5];
                        __syncwarp();
                        if (!((sw >> (Sb & 31)) & 1u)) coop_down_or(st, 1, Sb, 0u, lane);
                        if (Lb != Sb) {
                            uint32_t *tr = TIES ? st + G::WB : tie32 + (jt >> 5) * (G::WB * 32) + (jt & 31);
                            coop_down_or(tr, TIES ? 1 : 32, Lb, Lb & ~Sb, lane);
                        }
                    }
                    __syncwarp();
#endif
                }
        };
        int qn = 0;
        uint32_t npair32 = 0;
        for (int g = 0; g < ngroups; g++) {
            const uint32_t nw = use_super ? need[g] : 0xffffffffu;
            if (nw == 0) continue;
            const int tt = min(g * 32 + lane, nt - 1);
            uint32_t le[G::CW];
#pragma unroll
            for (int k = 0; k < G::CW; k++) le[k] = pH[tt * CWP + k] - mn[k];  // guard <=> corner <= p
            const uint32_t Mb = gather_mask<G::NG>(le);
            const uint32_t wb = state[tt * C::PS + (Mb >> 5)];
            const bool needp = ((nw >> lane) & 1u) && g * 32 + lane < nt && !(__funnelshift_r(wb, wb, Mb) & 1u);
            const uint32_t todo = __ballot_sync(0xffffffffu, needp);
            if (use_super) n_box += __popc(nw);
            if (todo == 0) continue;
            npair32 += __popc(todo);
            if (needp) wq[qn + __popc(todo & ((1u << lane) - 1u))] = g * 32 + lane;
            qn += __popc(todo);
            __syncwarp();
            while (qn >= kCU) {
                qn -= kCU;
                int ts[kCU];
#pragma unroll
                for (int u = 0; u < kCU; u++) ts[u] = wq[qn + u];
                run_batch(ts, kCU);
            }
            __syncwarp();
        }
        if (qn > 0) {
            int ts[kCU];
#pragma unroll
            for (int u = 0; u < kCU; u++) ts[u] = wq[min(u, qn - 1)];
            run_batch(ts, qn);
        }
        if (!use_super) n_box += nt;
        n_pair += 32ull * npair32;
    }
    if (counters) {
        if (lane == 0) {
            atomicAdd(&counters[2], n_box);
            atomicAdd(&counters[3], n_pair);
        }
        for (int o = 16; o; o >>= 1) n_miss += __shfl_xor_sync(0xffffffffu, n_miss, o);
        if (lane == 0) atomicAdd(&counters[4], n_miss);
    }
    asm volatile("bar.sync 1, %0;" ::"r"(kCWarps * 32) : "memory");
    for (int t = warp; t < nt; t += kCWarps) {
        const int64_t jt = j0 + t;
        const uint32_t *st = state + t * C::PS;
        uint32_t *out = rows32 + (jt >> 5) * (G::WB * 32) + (jt & 31);
        const uint32_t *trg = tie32 + (jt >> 5) * (G::WB * 32) + (jt & 31);
        for (int w = lane; w < G::WB; w += 32) {
            uint32_t v;
            if (MODE == kModeDims) {  // p dominated in delta <=> delta in D_i for some i in delta
                v = 0;
#pragma unroll
                for (int i = 0; i < D; i++) {
                    const uint32_t in = i < 5 ? low_dim_pattern(i) : (((w >> (i - 5)) & 1u) ? 0xffffffffu : 0u);
                    v |= st[(1 + i) * G::WB + w] & in;
                }
            } else {
                v = st[w] | (TIES ? st[G::WB + w] : trg[w * 32]);
            }
            uint32_t row = ~v & G::kRowMask;
            if (w == 0) row &= ~1u;
            out[w * 32] = row;
            if (ext_rows32) {
                uint32_t er = ~st[w] & G::kRowMask;
                if (w == 0) er &= ~1u;
                ext_rows32[(jt >> 5) * (G::WB * 32) + w * 32 + (jt & 31)] = er;
            }
        }
    }
}

// Super-chunk (tile corner) phase of design C: off by default — on the anticorrelated workloads the tile
// corner almost never prunes and the per-tile consumer barrier costs 40% (H: 147 -> 206 ms); on tie-heavy
// data (C5) it removes 92% of the chunk tests at equal time.  SKYCUBE_K3_SUPER=1 enables it (A/B runs).
inline int super_enabled() {
    const char *e = getenv("SKYCUBE_K3_SUPER");
    return e && e[0] == '1';
}

template <int D, int MODE>
void launch_c_t(Ctx &c, int64_t j_begin, int64_t j_end, uint32_t *rows32, uint32_t *ext_rows32, cudaStream_t st) {
    using G = Geo<D>;
    using C = GeoC<D, MODE>;
    // tasks per CTA: the shared-memory budget, but at least one CTA per SM for small ranges
    const int64_t range = j_end - j_begin;
    const int tpc = (int)std::min<int64_t>(C::NT, std::max<int64_t>(32, ceil_div(ceil_div(range, c.num_sms), 32) * 32));
    const size_t smem = sizeof(uint32_t) * (4 * kCStages + (size_t)kCStages * C::TW +
                                            (size_t)tpc * (((G::CW + 3) & ~3) + (G::CW | 1)) + (size_t)tpc * C::PS +
                                            (size_t)tpc + 2 * (size_t)ceil_div(tpc, 32) + kCWarps * 128);
    SKY_CUDA(cudaFuncSetAttribute(k3_mdmc_c_kernel<D, MODE>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    const unsigned blocks = (unsigned)ceil_div(range, tpc);
    k3_mdmc_c_kernel<D, MODE><<<blocks, (kCWarps + 1) * 32, smem, st>>>(
        c.p_codes.as<uint32_t>(), c.p_ord.as<uint32_t>(), c.chunks_ext.as<uint32_t>(), c.q_ord.as<uint32_t>(),
        c.minord.as<uint32_t>(), c.supers_ext.as<uint32_t>(), super_enabled(), c.nchunks_ext, j_begin, j_end, ~c.exact_mask & ((1u << D) - 1u), tpc, rows32, c.tie.as<uint32_t>(), ext_rows32,
        c.counters.as<unsigned long long>());
    c.L.count++;
    SKY_LAUNCH_CHECK();
}

// Tie-heavy inputs (every dimension discrete enough for injective codes) or small d: the tie-exact state
// (kModeDims, d <= 12) unless B_{p notin S+} itself is requested (ext rows), then kModeSmemTie.  Continuous
// data at d > 10: ties are rare and go to a global row (kModeGlobalTie).
template <int D>
void launch_c(Ctx &c, int64_t j_begin, int64_t j_end, uint32_t *rows32, uint32_t *ext_rows32, cudaStream_t st) {
    const bool all_exact = c.exact_mask == ((1u << D) - 1u);
    const char *m = getenv("SKYCUBE_K3_MODE");  // test hook: force a state mode
    int mode = (D <= 10 || all_exact) ? (D <= 12 && !ext_rows32 ? kModeDims : kModeSmemTie) : kModeGlobalTie;
    if (m && *m) {
        mode = m[0] - '0';
        if (mode == kModeDims && (D > 12 || ext_rows32)) mode = kModeSmemTie;
    }
    if (mode == kModeDims) {
        if constexpr (D <= 12) launch_c_t<D, kModeDims>(c, j_begin, j_end, rows32, ext_rows32, st);
    } else if (mode == kModeSmemTie) {
        launch_c_t<D, kModeSmemTie>(c, j_begin, j_end, rows32, ext_rows32, st);
    } else {
        launch_c_t<D, kModeGlobalTie>(c, j_begin, j_end, rows32, ext_rows32, st);
    }
}

template <int D, bool TIES>
void launch_a_t(Ctx &c, int64_t j_begin, int64_t j_end, uint32_t *rows32, uint32_t *ext_rows32, cudaStream_t st) {
    using G = Geo<D>;
    const size_t smem = sizeof(uint32_t) * (4 * kAStages + kAStages * (size_t)kATQ * G::CW +
                                            (TIES ? 2 : 1) * (size_t)kAWarps * G::WB * 32);
    SKY_CUDA(cudaFuncSetAttribute(k3_mdmc_a_kernel<D, TIES>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    const int64_t ntq = ceil_div(c.m, kATQ);
    const unsigned blocks = (unsigned)ceil_div(j_end - j_begin, kAWarps * 32);
    k3_mdmc_a_kernel<D, TIES><<<blocks, (kAWarps + 1) * 32, smem, st>>>(
        c.p_codes.as<uint32_t>(), c.p_ord.as<uint32_t>(), c.q_codes.as<uint32_t>(), c.q_ord.as<uint32_t>(), ntq,
        j_begin, j_end, ~c.exact_mask & ((1u << D) - 1u), rows32, c.tie.as<uint32_t>(), ext_rows32);
    c.L.count++;
    SKY_LAUNCH_CHECK();
}

// Tie-heavy inputs (every dimension discrete enough for injective codes) or small d keep the tie part of
// B_{p notin S} in shared memory; otherwise ties are rare and go to a global row.
template <int D>
void launch_a(Ctx &c, int64_t j_begin, int64_t j_end, uint32_t *rows32, uint32_t *ext_rows32, cudaStream_t st) {
    const bool all_exact = c.exact_mask == ((1u << D) - 1u);
    if (D <= 10 || all_exact) launch_a_t<D, true>(c, j_begin, j_end, rows32, ext_rows32, st);
    else launch_a_t<D, false>(c, j_begin, j_end, rows32, ext_rows32, st);
}

template <int D>
void launch_b(Ctx &c, int64_t j_begin, int64_t j_end, uint32_t *rows32, uint32_t *ext_rows32, cudaStream_t st) {
    using G = Geo<D>;
    constexpr int NT = GeoB<D>::NT;
    const size_t smem = sizeof(uint32_t) * (4 * kBStages + kBStages * (size_t)kBTQ * G::CW + (size_t)NT * G::CW +
                                            (size_t)NT * G::WB);
    SKY_CUDA(cudaFuncSetAttribute(k3_mdmc_b_kernel<D>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    const int64_t ntq = ceil_div(c.m, kBTQ);
    const unsigned blocks = (unsigned)ceil_div(j_end - j_begin, NT);
    k3_mdmc_b_kernel<D><<<blocks, (kBWarps + 1) * 32, smem, st>>>(
        c.p_codes.as<uint32_t>(), c.p_ord.as<uint32_t>(), c.q_codes.as<uint32_t>(), c.q_ord.as<uint32_t>(), ntq,
        j_begin, j_end, ~c.exact_mask & ((1u << D) - 1u), rows32, c.tie.as<uint32_t>(), ext_rows32);
    c.L.count++;
    SKY_LAUNCH_CHECK();
}

// Competitor stream padded to whole tiles with "never better" points (code 0x7fff, key 0xffffffff).
__global__ void pad_q_kernel(uint32_t *q_codes, uint32_t *q_ord, int64_t m, int64_t mpad, int cw, int d) {
    const int64_t q = m + (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (q >= mpad) return;
    for (int k = 0; k < cw; k++) q_codes[q * cw + k] = 0x7fff7fffu;
    for (int i = 0; i < d; i++) q_ord[q * d + i] = 0xffffffffu;
}

}  // namespace

void mdmc_run(Ctx &c, int64_t j_begin, int64_t j_end, uint32_t *d_rows32, uint32_t *d_ext_rows32, cudaStream_t st) {
    if (!c.ext_ready) throw Error{1, "skycube_dev_mdmc before skycube_dev_set_ext"};
    if (j_begin < 0 || j_end > c.m || (j_begin & 31)) throw Error{1, "bad MDMC task range"};
    if (j_end <= j_begin) return;
    const int d = c.d;
    const int cw = c.dp / 2;
    // q stream padding to whole tiles (both designs use tiles of at most 256)
    const int64_t mpad = ceil_div(c.m, kQPad) * kQPad;  // capacity reserved by ext_build
    if (mpad > c.m) {
        pad_q_kernel<<<(unsigned)ceil_div(mpad - c.m, 256), 256, 0, st>>>(c.q_codes.as<uint32_t>(), c.q_ord.as<uint32_t>(),
                                                                          c.m, mpad, cw, d);
        c.L.count++;
        SKY_LAUNCH_CHECK();
    }
    const int64_t g0 = j_begin >> 5, g1 = ceil_div(j_end, 32);
    const size_t grp_words = (size_t)c.W * 32;
    c.tie.ensure(sizeof(uint32_t) * grp_words * (size_t)ceil_div(c.m, 32));
    SKY_CUDA(cudaMemsetAsync(c.tie.as<uint32_t>() + g0 * grp_words, 0, sizeof(uint32_t) * grp_words * (g1 - g0), st));
    const char *sel = getenv("SKYCUBE_K3");
    const char design = sel && *sel ? sel[0] : 'c';
    if (design == 'c') {
        switch (d) {
#define SKY_C(DD) case DD: launch_c<DD>(c, j_begin, j_end, d_rows32, d_ext_rows32, st); break;
            SKY_C(1) SKY_C(2) SKY_C(3) SKY_C(4) SKY_C(5) SKY_C(6) SKY_C(7) SKY_C(8)
            SKY_C(9) SKY_C(10) SKY_C(11) SKY_C(12) SKY_C(13) SKY_C(14) SKY_C(15) SKY_C(16)
#undef SKY_C
            default: throw Error{1, "d must be in [1, 16]"};
        }
        return;
    }
    switch (d) {
        case 1: launch_a<1>(c, j_begin, j_end, d_rows32, d_ext_rows32, st); break;
        case 2: launch_a<2>(c, j_begin, j_end, d_rows32, d_ext_rows32, st); break;
        case 3: launch_a<3>(c, j_begin, j_end, d_rows32, d_ext_rows32, st); break;
        case 4: launch_a<4>(c, j_begin, j_end, d_rows32, d_ext_rows32, st); break;
        case 5: launch_a<5>(c, j_begin, j_end, d_rows32, d_ext_rows32, st); break;
        case 6: launch_a<6>(c, j_begin, j_end, d_rows32, d_ext_rows32, st); break;
        case 7: launch_a<7>(c, j_begin, j_end, d_rows32, d_ext_rows32, st); break;
        case 8: launch_a<8>(c, j_begin, j_end, d_rows32, d_ext_rows32, st); break;
        case 9: launch_a<9>(c, j_begin, j_end, d_rows32, d_ext_rows32, st); break;
        case 10: launch_a<10>(c, j_begin, j_end, d_rows32, d_ext_rows32, st); break;
        case 11: launch_a<11>(c, j_begin, j_end, d_rows32, d_ext_rows32, st); break;
        case 12: launch_a<12>(c, j_begin, j_end, d_rows32, d_ext_rows32, st); break;
        case 13: launch_b<13>(c, j_begin, j_end, d_rows32, d_ext_rows32, st); break;
        case 14: launch_b<14>(c, j_begin, j_end, d_rows32, d_ext_rows32, st); break;
        case 15: launch_b<15>(c, j_begin, j_end, d_rows32, d_ext_rows32, st); break;
        case 16: launch_b<16>(c, j_begin, j_end, d_rows32, d_ext_rows32, st); break;
        default: throw Error{1, "d must be in [1, 16]"};
    }
}

}  // namespace sky
