// k3_mdmc.cu — K3: the MDMC per-point task of Alg. 3 (L318-324), lines 3-12, on sm_100a.
//
// For every p in S+(P) (the data-parallel tasks, L308-310) and every competitor q in S+(P) (Λ1:
// competitors outside S+ add nothing), the pair reduces to two d-bit masks (L82)
//     L = B_{q<=p},  S = B_{q<p}   (E = L \ S = B_{q=p})
// and q dominates p exactly in the subspaces { delta subset of L : delta & S != 0 } (Def. 1), strictly in the
// non-empty subsets of S.  B_{p notin S+} (strict) is downward closed, so bit L set in it means q adds
// nothing new (L330-336, Alg. 3 line 11) — the probe that skips almost every pair.
//
// Competitors are S+ in static-tree (Morton) order, in chunks of 32 with their lower corner, visited
// strongest corner first (prep.cu).  For a task p and a chunk, Mbox = B_{corner<=p} is a superset of M(q,p)
// for every q of the chunk, so bit Mbox set in the probe set proves the whole chunk adds nothing (Λ4 on a
// leaf range: the paper's filter on path labels, L446-452, with the tree's global pivots).
//
// Design A (k3_mdmc_kernel): a CTA holds up to NT tasks (codes + state in shared memory) and streams every
// chunk once (TMA ring fed by one producer warp); each of the 16 consumer warps takes one chunk per tile, one
// competitor per lane in registers.  Design O (k3_owner_kernel, further below) swaps the roles: a warp owns
// 32 tasks and takes a share of every tile's chunks.  Both run the same three passes:
//   box pass   lane l tests task 32g+l against the chunk corner (SWAR over 16-bit code lanes with guard
//              bits, gathered to a d-bit mask with a byte permute and a carry-free multiply per 4
//              dimensions) and probes the task's state; a ballot gives the tasks whose chunk must be opened;
//   sub pass   opened tasks, 4 at a time: lane (u, s) tests task u against the corner of sub-chunk s (4
//              points, the level below); opened (task, sub-chunk) items are queued;
//   pair pass  8 items at a time: lane (k, r) takes member r of item k's sub-chunk (shuffled from the lane
//              that holds it) and forms M = B_{code(q)<=code(p)} (a superset of L: codes are monotone, Λ3),
//              then probes bit M; set => skip (Λ4);
//   miss       (rare: ~0.3% of pair tests on the anticorrelated headline) the lane computes the exact L, S
//              (strict SWAR compare plus exact keys on tied, non-injective codes); then the whole warp
//              expands each contributing competitor word-parallel (Alg. 3 line 12: for the word index w, the
//              high bits of delta, OR in the pattern of the subsets of the low 5 bits; lanes split the words).
//
// Per-task state modes (shared memory):
//   kModeGlobalTie  B_{p notin S+} is the probe set; the tie part of B_{p notin S} (reading Q3) goes to a
//                   global row (continuous data at d > 10: ties are rare).
//   kModeSmemTie    B_{p notin S+} and the tie part, both in shared memory (tie-heavy / d <= 10 when the
//                   B_{p in S+} rows themselves are requested).
//   kModeDims       tie-exact state (d <= 12, tie-heavy or low d): one downward-closed set per dimension,
//                   D_i = union of sub(L_q) over the q with i in S_q, and the probe set
//                   K = { delta : delta in D_i for every i in delta \ Z_p } (Z_p: dimensions where p holds the
//                   global minimum, so no q is strictly better there).  p is dominated in delta <=> delta in D_i
//                   for some i in delta (Def. 1), and bit M in K proves that q (S_q subset of L_q \ Z_p,
//                   L_q subset of M) adds nothing to any D_i.  Without ties K is B_{p notin S+}; under ties
//                   it keeps growing where B_{p notin S+} cannot (ties at the optimum): C5 misses 19K -> 30
//                   per task.
// The result is scheduling-independent (every update is an OR of a correct contribution, every skip is
// sound for any subset of the final state), so racing warps and any chunk order give identical bytes.
#include <algorithm>

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

constexpr int kWarps = 16;                // consumer warps = chunks per tile (+1 producer warp)
// TMA ring depth: 4 stages; at d >= 15 the 2^d-bit task state crowds shared memory (8 KB per task at d = 16),
// and two stages buy 5 more tasks per CTA (19 -> 24)
#ifndef SKY_K3_STAGES
#define SKY_K3_STAGES 4
#endif
#ifndef SKY_K3_STAGES_WIDE
#define SKY_K3_STAGES_WIDE 2  // ring stages of the 24-warp (24-chunk tile) kernel: 2 measured better than 3
                              // (C3A K3 35.6 -> 34.0 ms: more tasks per CTA; H 87.1 -> 86.7)
#endif
#ifndef SKY_K3_STAGES_HIGHD
#define SKY_K3_STAGES_HIGHD 2
#endif
template <int D>
constexpr int k3_stages() { return D >= 15 ? SKY_K3_STAGES_HIGHD : SKY_K3_STAGES; }
constexpr int kSmemBytes = 227 * 1024;    // opt-in maximum per CTA
constexpr int kModeGlobalTie = 0, kModeSmemTie = 1, kModeDims = 2;
static_assert(kWarps == kTileChunks, "one chunk per consumer warp per tile");

template <int D, int MODE, int NW = kWarps, int ST = 0>
struct GeoK3 {
    static constexpr int PER = (MODE == kModeGlobalTie ? 1 : MODE == kModeSmemTie ? 2 : D + 1) * Geo<D>::WB;
    static constexpr int PS = PER | 1;                                   // odd task stride (bank spread)
    static constexpr int CWV = (Geo<D>::CW + 3) & ~3;                    // 16-byte code stride (pair pass)
    static constexpr int REC = 32 * Geo<D>::CW + kCoarseRows * kCoarseWords;  // chunk record words (ctx.cuh)
    static constexpr int CO = 32 * Geo<D>::CW;                           // coarse chunk corner; sub-corner s at CO+4+4s
    static constexpr int TW = NW * REC;                                  // tile words (one chunk per consumer warp)
    static constexpr int kStages = ST > 0 ? ST : NW > kWarps && D < 15 ? SKY_K3_STAGES_WIDE : k3_stages<D>();
    static constexpr int RING = 4 * kStages + kStages * TW;              // barriers + stages (words)
    static constexpr int QW = 96;                                        // per-warp queue words (tasks, items)
    static constexpr int ROW = PS + kCoarseWords + CWV + 1;              // words per task: state, coarse, fine, Z_p
    static constexpr int NT0 = (kSmemBytes / 4 - RING - NW * QW - 64) / ROW;
    static constexpr int NT = NT0 < 1024 ? NT0 : 1024;                   // tasks per CTA
    static size_t smem_bytes(int tpc) { return sizeof(uint32_t) * ((size_t)RING + (size_t)tpc * ROW + NW * QW); }
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

// Coarse corner test (chunk records, ctx.cuh): 7-bit codes, four dimensions per word (byte k = dimension 4g+k),
// the task side carrying a guard bit per byte: x = (p | 0x80808080) - corner has the guard bit of byte k set
// <=> corner_k <= p_k (no borrow crosses a byte).  Word g -> mask bits 4g..4g+3 by the same carry-free multiply.
template <int NQ>
__device__ __forceinline__ uint32_t gather_coarse(const uint32_t *x) {
    uint32_t m = 0;
#pragma unroll
    for (int g = NQ - 1; g >= 0; g--) m = __funnelshift_l((x[g] & 0x80808080u) * 0x00204081u, m, 4);
    return m;
}

// The coarse code row of task t (four words, guard bits set) from its fine 15-bit code words; dimensions >= D are 0.
template <int D, int CW>
__device__ __forceinline__ void coarse_row(const uint32_t *fine, uint64_t cshift, uint32_t *out) {
#pragma unroll
    for (int g = 0; g < kCoarseWords; g++) {
        uint32_t w = 0x80808080u;
#pragma unroll
        for (int b = 0; b < 4; b++) {
            const int i = 4 * g + b;
            if (i < D) {
                const uint32_t code = (fine[i >> 1] >> (16 * (i & 1))) & 0x7fffu;
                w |= min(code >> ((cshift >> (4 * i)) & 15u), 127u) << (8 * b);
            }
        }
        out[g] = w;
    }
}

// Bits delta_low (0..31) that are subsets of x (x < 32): the word pattern of sub(x) in the low 5 dims.
// the same as a table (warp-uniform index: one constant-cache load instead of ~10 instructions)
__constant__ uint32_t kSub5[32] = {
    0x00000001u, 0x00000003u, 0x00000005u, 0x0000000fu, 0x00000011u, 0x00000033u, 0x00000055u, 0x000000ffu,
    0x00000101u, 0x00000303u, 0x00000505u, 0x00000f0fu, 0x00001111u, 0x00003333u, 0x00005555u, 0x0000ffffu,
    0x00010001u, 0x00030003u, 0x00050005u, 0x000f000fu, 0x00110011u, 0x00330033u, 0x00550055u, 0x00ff00ffu,
    0x01010101u, 0x03030303u, 0x05050505u, 0x0f0f0f0fu, 0x11111111u, 0x33333333u, 0x55555555u, 0xffffffffu};

__device__ __forceinline__ uint32_t sub5(uint32_t x) {
    uint32_t t = 1u;
    if (x & 1u) t |= t << 1;
    if (x & 2u) t |= t << 2;
    if (x & 4u) t |= t << 4;
    if (x & 8u) t |= t << 8;
    if (x & 16u) t |= t << 16;
    return t;
}

// Word pattern of the low-5-bit subspaces that contain dimension i (i < 5).
__device__ __forceinline__ uint32_t low_dim_pattern(int i) {
    return i == 0 ? 0xaaaaaaaau : i == 1 ? 0xccccccccu : i == 2 ? 0xf0f0f0f0u : i == 3 ? 0xff00ff00u : 0xffff0000u;
}

// Word pattern of the subspaces of word w that contain dimension i.
__device__ __forceinline__ uint32_t dim_in_word(int i, uint32_t w) {
    return i < 5 ? low_dim_pattern(i) : (((w >> (i - 5)) & 1u) ? 0xffffffffu : 0u);
}

// Exact B_{q<=p}, B_{q<p}: the strict SWAR compare, then the exact keys on the dimensions whose codes tie
// but are not injective (M is B_{code(q)<=code(p)}).
template <int D>
__device__ __forceinline__ void exact_masks(const uint32_t *ph, const uint32_t *q, uint32_t M, uint32_t inexact,
                                            const uint32_t *__restrict__ qo, const uint32_t *__restrict__ po,
                                            uint32_t &L, uint32_t &S) {
    using G = Geo<D>;
    uint32_t lt[G::CW];
#pragma unroll
    for (int k = 0; k < G::CW; k++) lt[k] = ph[k] - q[k] - 0x00010001u;  // guard <=> code(q) < code(p)
    S = gather_mask<G::NG>(lt);
    L = M;
    uint32_t U = M & ~S & inexact;
    while (U) {
        const int i = __ffs(U) - 1;
        U &= U - 1;
        const uint32_t qv = qo[i], pv = po[i];
        if (qv > pv) L &= ~(1u << i);
        else if (qv < pv) S |= 1u << i;
    }
}

// Shared-memory word access through a 32-bit shared-window address computed once per kernel.  Plain
// pointer accesses made the compiler re-materialise the dynamic shared base (S2UR SR_CgaCtaId + ULEA) in
// the hot loops.  Probes are volatile: other warps OR bits into the state concurrently (any value read
// is a sound subset of the final state).
__device__ __forceinline__ uint32_t lds_u32(uint32_t a) {
    uint32_t v;
    asm volatile("ld.shared.u32 %0, [%1];" : "=r"(v) : "r"(a));
    return v;
}
__device__ __forceinline__ void sts_u32(uint32_t a, uint32_t v) { asm volatile("st.shared.u32 [%0], %1;" ::"r"(a), "r"(v) : "memory"); }
// (laundered through an opaque move, or the compiler re-derives it from SR_CgaCtaId at every use)
__device__ __forceinline__ uint32_t smem_addr(const void *p) {
    uint32_t a = (uint32_t)__cvta_generic_to_shared(p);
    asm volatile("mov.b32 %0, %0;" : "+r"(a));
    return a;
}

__device__ __forceinline__ void red_or_s(uint32_t a, uint32_t v) { asm volatile("red.shared.or.b32 [%0], %1;" ::"r"(a), "r"(v) : "memory"); }
__device__ __forceinline__ void exch_s(uint32_t a, uint32_t v) {
    uint32_t old;
    asm volatile("atom.shared.exch.b32 %0, [%1], %2;" : "=r"(old) : "r"(a), "r"(v) : "memory");
}

// kModeGlobalTie: the tie rows are zeroed before the kernel (memset) and a task's row is marked in shared memory
// (flag 2) when a tie is first OR-ed into it; the epilogue reads only marked rows.  Ties are rare in the
// continuous data this mode runs on, so the epilogue's read-back of 8 KB per task at d = 16 disappears (C4:
// 7.3 GB of the 15.4 GB of DRAM traffic per K3 launch in round 1).  (Zeroing the rows lazily in the kernel
// instead of the memset lost tie bits to a race -- tests/test_gpu_parity.py::test_global_tie_rows_d16 --
// and was dropped.)
__device__ __forceinline__ void tie_row_mark(uint32_t flag_s, int lane) {
    if (lane == 0) exch_s(flag_s, 2u);
}

// Warp-cooperative walk over the state words whose word index w (the subspace's dimensions 5..d-1) is a subset
// of H.  Up to 8 words per lane (d <= 13): every lane tests its words w = lane + 32k directly (no subset
// arithmetic, no loop-carried state; C5 K3 29.5 -> 26.8 ms, C3A 39.4 -> 38.9).  Above (up to 2048 words): the
// lanes take the subsets of the lowest five set bits of H (the lane index deposited into them), each lane
// walks the subsets of the remaining bits -- all 32 lanes busy whatever H is.  (A fixed split -- lane = the
// low five bits of w -- leaves most lanes idle when H has few low bits: C4 K3 660 -> 702 ms.)
template <int WB, class F>
__device__ __forceinline__ void coop_words(uint32_t H, int lane, F &&f) {
    if constexpr (WB <= 256) {
#pragma unroll
        for (int k = 0; k < (WB + 31) / 32; k++) {
            const uint32_t w = (uint32_t)lane + 32u * k;
            if ((WB % 32 == 0 || w < (uint32_t)WB) && (w & ~H) == 0u) f(w);
        }
    } else {
        uint32_t rest = H, w_lo = 0;
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
                f(w_lo | w_hi);
                w_hi = (w_hi - rest) & rest;
            } while (w_hi);
        }
    }
    __syncwarp();
}

// Alg. 3 line 12 for one contributing competitor (S != 0), the whole warp: st_s = shared address of the task's
// state, L and S exact; tie_g = the task's global tie row (kModeGlobalTie, word stride 32), else unused.
// Atomic ORs (red.shared / red.global): other warps update the same task concurrently.
template <int D, int MODE>
__device__ __forceinline__ void expand(uint32_t st_s, uint32_t *tie_g, uint32_t tflag_s, uint32_t L, uint32_t S, uint32_t z,
                                       int lane) {
    using G = Geo<D>;
    constexpr int WB = G::WB;
    const uint32_t lh = L >> 5, lb = kSub5[L & 31u];
    if (MODE == kModeDims) {
        bool changed = false;  // warp-uniform
        for (uint32_t s = S; s; s &= s - 1) {  // D_i |= sub(L) for every i in S
            const uint32_t Di = st_s + 4u * (1 + (__ffs(s) - 1)) * WB;
            if ((lds_u32(Di + 4u * lh) >> (L & 31)) & 1u) continue;  // downward closed: sub(L) already there
            changed = true;
            coop_words<WB>(lh, lane, [&](uint32_t w) { red_or_s(Di + 4u * w, lb); });
        }
        if (!changed) return;
        // K on the words of sub(L) (only there can D change).  Racing warps may compute K from stale D words:
        // that only leaves K smaller (still sound); bits are only ever OR-ed in.
        coop_words<WB>(lh, lane, [&](uint32_t w) {
            uint32_t k = 0xffffffffu;
#pragma unroll
            for (int i = 0; i < D; i++)
                if (!((z >> i) & 1u)) k &= lds_u32(st_s + 4u * ((1 + i) * WB + w)) | ~dim_in_word(i, w);
            red_or_s(st_s + 4u * w, k);
        });
        return;
    }
    // B_{p notin S+} |= sub(S) (strict dominance propagates), unless already there
    if (!((lds_u32(st_s + 4u * (S >> 5)) >> (S & 31)) & 1u)) {
        const uint32_t sb = kSub5[S & 31u];
        coop_words<WB>(S >> 5, lane, [&](uint32_t w) { red_or_s(st_s + 4u * w, sb); });
    }
    if (L == S) return;
    // ties: B_{p notin S} |= sub(L) \ sub(E), E = B_{q=p}  (reading Q3)
    const uint32_t E = L & ~S, eh = E >> 5, eb = kSub5[E & 31u];
    if (MODE == kModeGlobalTie) tie_row_mark(tflag_s, lane);
    coop_words<WB>(lh, lane, [&](uint32_t w) {
        const uint32_t bits = (w & ~eh) ? lb : (lb & ~eb);
        if (bits) {
            if (MODE == kModeSmemTie) red_or_s(st_s + 4u * (WB + w), bits);
            else atomicOr(&tie_g[w * 32], bits);
        }
    });
}

// Partial skycube (Appendix A.2; reading P1): bits b of a membership word whose subspace
// 32w + b has at most k dimensions in the low five (k = d' - |w|, w the word index = dimensions 5..d-1).
__device__ __forceinline__ uint32_t level_pattern(int k) {
    if (k < 0) return 0u;
    uint32_t r = 0;
#pragma unroll
    for (int b = 0; b < 32; b++)
        if (__popc(b) <= k) r |= 1u << b;
    return r;
}

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

// The same from a 32-bit shared address (read-only task codes: plain asm, free to schedule).
template <int CW>
__device__ __forceinline__ void load_row_s(uint32_t a, uint32_t *w) {
#pragma unroll
    for (int k = 0; k + 4 <= CW; k += 4)
        asm("ld.shared.v4.u32 {%0, %1, %2, %3}, [%4];"
            : "=r"(w[k]), "=r"(w[k + 1]), "=r"(w[k + 2]), "=r"(w[k + 3])
            : "r"(a + 4u * k));
    if (CW % 4) asm("ld.shared.v2.u32 {%0, %1}, [%2];" : "=r"(w[CW & ~3]), "=r"(w[(CW & ~3) + 1]) : "r"(a + 4u * (CW & ~3)));
}

// Epilogue of both K3 designs: B_{p notin S} -> membership row (its complement; bit 0, the empty subspace,
// is never a member), written in the tiled layout (group of 32 tasks, word-major).
template <int D, int MODE, int NW = kWarps>
__device__ __forceinline__ void write_rows(const uint32_t *state, int64_t j0, int nt, int warp, int lane, int max_level,
                                           uint32_t *__restrict__ rows32, const uint32_t *__restrict__ tie32,
                                           uint32_t *__restrict__ ext_rows32, uint32_t *__restrict__ host_mem,
                                           const int32_t *__restrict__ ext_ids, const uint32_t *tflag) {
    using G = Geo<D>;
    using C = GeoK3<D, MODE>;
    constexpr bool TIES = MODE == kModeSmemTie;
    for (int t = warp; t < nt; t += NW) {
        const int64_t jt = j0 + t;
        const uint32_t *st = state + t * C::PS;
        uint32_t *out = rows32 + (jt >> 5) * (G::WB * 32) + (jt & 31);
        const uint32_t *trg = tie32 + (jt >> 5) * (G::WB * 32) + (jt & 31);
        // zero-copy: the row also goes straight to the caller's pinned host membership array (by point id),
        // so its PCIe transfer overlaps the rest of the kernel instead of following the whole build
        uint32_t *hrow = host_mem ? host_mem + (int64_t)ext_ids[jt] * G::WB : nullptr;
        const bool tie_used = MODE == kModeGlobalTie && tflag[t] == 2u;
        for (int w = lane; w < G::WB; w += 32) {
            uint32_t v;
            if (MODE == kModeDims) {  // p dominated in delta <=> delta in D_i for some i in delta
                v = 0;
#pragma unroll
                for (int i = 0; i < D; i++) v |= st[(1 + i) * G::WB + w] & dim_in_word(i, w);
            } else {
                // tie rows are read from L2 (ld.global.cg): they were written by atomics during this kernel
                v = st[w] | (TIES ? st[G::WB + w] : tie_used ? __ldcg(&trg[w * 32]) : 0u);
            }
            const uint32_t lvl = max_level > 0 ? level_pattern(max_level - __popc(w)) : 0xffffffffu;
            uint32_t row = ~v & G::kRowMask & lvl;
            if (w == 0) row &= ~1u;
            out[w * 32] = row;
            if (hrow) hrow[w] = row;
            if (ext_rows32) {
                uint32_t er = ~st[w] & G::kRowMask & lvl;
                if (w == 0) er &= ~1u;
                ext_rows32[(jt >> 5) * (G::WB * 32) + w * 32 + (jt & 31)] = er;
            }
        }
    }
}

template <int D, int MODE, int NW>
__global__ void __launch_bounds__((NW + 1) * 32, 1) k3_mdmc_kernel(
    const uint32_t *__restrict__ p_codes, const uint32_t *__restrict__ p_ord, const uint32_t *__restrict__ chunks,
    const uint32_t *__restrict__ q_ord, const uint32_t *__restrict__ minord, int64_t nchunks, int64_t j_begin,
    int64_t j_end, uint32_t inexact, uint64_t cshift, int tpc, int max_level, uint32_t *__restrict__ rows32, uint32_t *__restrict__ tie32,
    uint32_t *__restrict__ ext_rows32, unsigned long long *__restrict__ counters, uint32_t *__restrict__ host_mem,
    const int32_t *__restrict__ ext_ids) {
    using G = Geo<D>;
    using C = GeoK3<D, MODE, NW>;
    constexpr int CWV = C::CWV, REC = C::REC, NQ = (D + 3) / 4;
    extern __shared__ __align__(128) uint32_t smem[];
    uint64_t *bars = reinterpret_cast<uint64_t *>(smem);
    constexpr int kStages = C::kStages;
    const TileRing<kStages> ring{bars, bars + kStages, smem + 4 * kStages, (uint32_t)C::TW};
    uint32_t *pV = smem + C::RING;             // [tpc][CWV] task codes with guard bits (pair pass)
    uint32_t *pC = pV + tpc * CWV;             // [tpc][4] coarse task codes with guard bits (corner tests)
    uint32_t *state = pC + tpc * kCoarseWords; // [tpc][PS]
    uint32_t *zm = state + tpc * C::PS;        // [tpc] Z_p (kModeDims)
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    uint32_t *wq = zm + tpc + warp * C::QW;    // per-warp queue of opened tasks (<= 3 + 32 entries)
    uint32_t *iq = wq + 40;                    // per-warp queue of opened (task, sub-chunk) items (<= 7 + 32)
    const uint32_t st_s = smem_addr(state), wq_s = smem_addr(wq), iq_s = smem_addr(iq), pV_s = smem_addr(pV);
    const uint32_t pC_s = smem_addr(pC);
    const uint32_t zm_s = smem_addr(zm);  // kModeGlobalTie: per-task tie-row flags (kModeDims: Z_p)
    const int64_t j0 = j_begin + (int64_t)blockIdx.x * tpc;
    const int nt = (int)min((int64_t)tpc, j_end - j0);
    const int64_t ntiles = ceil_div_dev(nchunks, NW);

    if (threadIdx.x == 0) ring.init(NW);
    for (int i = threadIdx.x; i < tpc * G::CW; i += blockDim.x) {
        const int t = i / G::CW, k = i % G::CW;
        uint32_t w = t < nt ? p_codes[(j0 + t) * G::CW + k] : 0u;
        if (2 * k >= D) w &= 0xffff0000u;  // padding dimensions: p = 0 never passes q <= p (q pad = 1)
        if (2 * k + 1 >= D) w &= 0x0000ffffu;
        pV[t * CWV + k] = w | kGuard;
    }
    __syncthreads();
    for (int t = threadIdx.x; t < tpc; t += blockDim.x) coarse_row<D, G::CW>(pV + t * CWV, cshift, pC + t * kCoarseWords);
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
        for (int t = threadIdx.x; t < tpc; t += blockDim.x) zm[t] = 0u;  // tie rows untouched
    }
    __syncthreads();
    if (warp == NW) {  // producer warp: one elected lane streams chunk tiles with TMA
        if (lane == 0)
            for (int64_t t = 0; t < ntiles; t++) ring.issue(chunks, t);
        return;
    }
    const int ngroups = (nt + 31) >> 5;
    unsigned long long n_box = 0, n_sub = 0, n_pair = 0, n_miss = 0, n_exp = 0;
    for (int64_t tile = 0; tile < ntiles; tile++) {
        ring.wait(tile);
        const uint32_t *rec = ring.stage(tile) + warp * REC;
        // this lane's competitor, the chunk's coarse corner, and the coarse corner of sub-chunk (lane & 7) — the
        // level below the chunk in the static tree (4 points) — all read before the stage is released
        uint32_t q[G::CW], mn[kCoarseWords], sc[kCoarseWords];
#pragma unroll
        for (int k = 0; k < G::CW; k++) q[k] = rec[lane * G::CW + k];
        load_row<kCoarseWords>(rec + C::CO, mn);
        load_row<kCoarseWords>(rec + C::CO + kCoarseWords * (1 + (lane & 7)), sc);
        // The loads above are still in flight (their values are first used much later): complete them before
        // the stage is handed back to the TMA producer, or the next tile's bulk copy can overwrite the stage
        // under them (observed as rare missing dominations at d >= 13 without this fence).
        __threadfence_block();
        __syncwarp();
        if (lane == 0) ring.release(tile);
        const int64_t c = tile * NW + warp;
        if (c >= nchunks) continue;

        // pair pass over packed items (task t, sub-chunk s): lane (k, r) = item k, member r of sub-chunk s; the
        // competitor comes from the lane that holds it (shuffle); misses run Alg. 3 lines 10-12 cooperatively
        auto pair_pass = [&](int base, int cnt) {
            const int k8 = lane >> 2, r = lane & 3;
            const uint32_t it = lds_u32(iq_s + 4u * (base + min(k8, cnt - 1)));
            const int t = (int)(it >> 3), src = (int)((it & 7u) << 2) + r;
            uint32_t qq[G::CW], x[G::CW];
#pragma unroll
            for (int k = 0; k < G::CW; k++) qq[k] = __shfl_sync(0xffffffffu, q[k], src);
            load_row_s<G::CW>(pV_s + 4u * (t * CWV), x);
#pragma unroll
            for (int k = 0; k < G::CW; k++) x[k] -= qq[k];  // guard <=> code(q) <= code(p)
            const uint32_t M = gather_mask<G::NG>(x);
            const uint32_t wd = lds_u32(st_s + 4u * (t * C::PS + (M >> 5)));
            const bool miss = k8 < cnt && !(__funnelshift_r(wd, wd, M) & 1u);
            if (!__any_sync(0xffffffffu, miss)) return;  // Λ4 for every lane
            uint32_t L = 0, S = 0;
            if (miss) {
                n_miss++;
                exact_masks<D>(pV + t * CWV, qq, M, inexact, q_ord + (c * 32 + src) * D, p_ord + (j0 + t) * D, L, S);
                if (S != 0 && L != M && ((lds_u32(st_s + 4u * (uint32_t)(t * C::PS + (L >> 5))) >> (L & 31)) & 1u))
                    S = 0;  // exact L covered
            }
            uint32_t todo = __ballot_sync(0xffffffffu, S != 0);
            n_exp += __popc(todo);
            while (todo) {
                const int from = __ffs(todo) - 1;
                todo &= todo - 1;
                const uint32_t Sb = __shfl_sync(0xffffffffu, S, from), Lb = __shfl_sync(0xffffffffu, L, from);
                const int tb = __shfl_sync(0xffffffffu, t, from);
                const int64_t jt = j0 + tb;
                expand<D, MODE>(st_s + 4u * (uint32_t)(tb * C::PS), tie32 + (jt >> 5) * (G::WB * 32) + (jt & 31),
                                zm_s + 4u * (uint32_t)tb, Lb, Sb, MODE == kModeDims ? zm[tb] : 0u, lane);
            }
        };

        // sub-chunk pass: lane (u, s) tests queued task u against sub-chunk corner s; the opened (task,
        // sub-chunk) items are queued and run 8 per pair pass
        int iqn = 0;
        uint32_t nsub32 = 0, nitem32 = 0;
        auto sub_pass = [&](int base, int cnt) {
            const int u = lane >> 3;
            const int t = (int)lds_u32(wq_s + 4u * (base + min(u, cnt - 1)));
            uint32_t x[kCoarseWords];
            load_row_s<kCoarseWords>(pC_s + 4u * (t * kCoarseWords), x);
#pragma unroll
            for (int k = 0; k < NQ; k++) x[k] -= sc[k];  // guard <=> coarse sub-corner <= p
            const uint32_t Ms = gather_coarse<NQ>(x);
            const uint32_t ws = lds_u32(st_s + 4u * (t * C::PS + (Ms >> 5)));
            const bool open = u < cnt && !(__funnelshift_r(ws, ws, Ms) & 1u);
            const uint32_t ob = __ballot_sync(0xffffffffu, open);
            nsub32 += 8 * cnt;
            if (!ob) return;
            nitem32 += __popc(ob);
            if (open) sts_u32(iq_s + 4u * (iqn + __popc(ob & ((1u << lane) - 1u))), ((uint32_t)t << 3) | (uint32_t)(lane & 7));
            iqn += __popc(ob);
            __syncwarp();
            while (iqn >= 8) {
                iqn -= 8;
                pair_pass(iqn, 8);
            }
            __syncwarp();
        };

        // box pass; the tasks whose chunk must be opened are pooled across task groups in a per-warp queue.
        // Two task groups per iteration: their mask chains and probes are independent (ILP).
        int qn = 0;
        auto enqueue = [&](uint32_t todo, int g) {
            if (todo == 0) return;
            if ((todo >> lane) & 1u) sts_u32(wq_s + 4u * (qn + __popc(todo & ((1u << lane) - 1u))), (uint32_t)(g * 32 + lane));
            qn += __popc(todo);
            __syncwarp();
            while (qn >= 4) {
                qn -= 4;
                sub_pass(qn, 4);
            }
            __syncwarp();
        };
        auto box_test = [&](int tt, uint32_t &Mb) {
            uint32_t le[kCoarseWords];
            load_row_s<kCoarseWords>(pC_s + 4u * (tt * kCoarseWords), le);  // one LDS.128: 4 conflict-free phases
#pragma unroll
            for (int k = 0; k < NQ; k++) le[k] -= mn[k];  // guard <=> coarse corner <= p
            Mb = gather_coarse<NQ>(le);
        };
        int g = 0;
        for (; g + 1 < ngroups; g += 2) {
            const int tt0 = g * 32 + lane, tt1 = min((g + 1) * 32 + lane, nt - 1);
            uint32_t Mb0, Mb1;
            box_test(tt0, Mb0);
            box_test(tt1, Mb1);
            const uint32_t wb0 = lds_u32(st_s + 4u * (tt0 * C::PS + (Mb0 >> 5)));
            const uint32_t wb1 = lds_u32(st_s + 4u * (tt1 * C::PS + (Mb1 >> 5)));
            const bool open0 = !(__funnelshift_r(wb0, wb0, Mb0) & 1u);
            const bool open1 = (g + 1) * 32 + lane < nt && !(__funnelshift_r(wb1, wb1, Mb1) & 1u);
            const uint32_t todo0 = __ballot_sync(0xffffffffu, open0), todo1 = __ballot_sync(0xffffffffu, open1);
            if ((todo0 | todo1) == 0) continue;
            enqueue(todo0, g);
            enqueue(todo1, g + 1);
        }
        if (g < ngroups) {  // odd group count (always the case at d >= 15: one group per CTA)
            const int tt = min(g * 32 + lane, nt - 1);
            uint32_t Mb;
            box_test(tt, Mb);
            const uint32_t wb = lds_u32(st_s + 4u * (tt * C::PS + (Mb >> 5)));
            enqueue(__ballot_sync(0xffffffffu, g * 32 + lane < nt && !(__funnelshift_r(wb, wb, Mb) & 1u)), g);
        }
        if (qn > 0) sub_pass(0, qn);
        if (iqn > 0) pair_pass(0, iqn);
        __syncwarp();
        n_sub += nsub32;
        n_pair += 4ull * nitem32;
        n_box += nt;
    }
    if (counters) {
        if (lane == 0) {
            atomicAdd(&counters[2], n_box);
            atomicAdd(&counters[3], n_pair);
        }
        for (int o = 16; o; o >>= 1) n_miss += __shfl_xor_sync(0xffffffffu, n_miss, o);
        if (lane == 0) {
            atomicAdd(&counters[4], n_miss);
            atomicAdd(&counters[5], n_sub);
            atomicAdd(&counters[6], n_exp);
        }
    }
    consumer_sync(NW * 32);
    write_rows<D, MODE, NW>(state, j0, nt, warp, lane, max_level, rows32, tie32, ext_rows32, host_mem, ext_ids, zm);
}


// CW words (CW even) from an 8-byte aligned shared address: the rows of a chunk record.
template <int CW>
__device__ __forceinline__ void load_row2_s(uint32_t a, uint32_t *w) {
#pragma unroll
    for (int k = 0; k < CW; k += 2) asm("ld.shared.v2.u32 {%0, %1}, [%2];" : "=r"(w[k]), "=r"(w[k + 1]) : "r"(a + 4u * k));
}

// ------------------------------------------------------------------------------------------------------
// Design O ("task owner", d <= 15): every consumer warp owns one group of 32 tasks (codes in registers, one
// task per lane) and a share of the chunks of every tile (wpg = 16 / groups warps per group split the 16
// chunks).  The chunk-corner test is then lane-parallel over tasks against a broadcast corner: no task-code
// reloads, no per-group loop.  Opened (task, chunk) items are queued and run through the same sub-chunk and
// pair passes as design A, reading the chunk's sub-corners and competitors from the ring stage, which the
// warp holds until it has finished the tile.  Needs 32 tasks' state in shared memory (d <= 15).
// design O's ring: 3 stages with 24 warps (a warp holds its stage until its sub/pair passes are done; C5 K3
// 20.6 ms with 2 stages, 20.2 with 3)
// (3 ring stages at d >= 15 too: the one partial group's 16 warps wait less at the tile boundary with a stage more
// of slack than they lose with one task fewer per CTA -- C4 K3 595.7 -> 576.6 ms; design A keeps 2 there)
#ifndef SKY_K3_O_STAGES_HIGHD
#define SKY_K3_O_STAGES_HIGHD 3
#endif
template <int D, int MODE, int NW>
using GeoO = GeoK3<D, MODE, NW, (D >= 15 ? SKY_K3_O_STAGES_HIGHD : NW > kWarps ? 3 : 0)>;

template <int D, int MODE, int NW>
__global__ void __launch_bounds__((NW + 1) * 32, 1) k3_owner_kernel(
    const uint32_t *__restrict__ p_codes, const uint32_t *__restrict__ p_ord, const uint32_t *__restrict__ chunks,
    const uint32_t *__restrict__ q_ord, const uint32_t *__restrict__ minord, int64_t nchunks, int64_t j_begin,
    int64_t j_end, uint32_t inexact, uint64_t cshift, int ngrp, int tpc, int max_level, uint32_t *__restrict__ rows32,
    uint32_t *__restrict__ tie32, uint32_t *__restrict__ ext_rows32, unsigned long long *__restrict__ counters,
    uint32_t *__restrict__ host_mem, const int32_t *__restrict__ ext_ids) {
    using G = Geo<D>;
    using C = GeoO<D, MODE, NW>;
    constexpr int CWV = C::CWV, REC = C::REC, NQ = (D + 3) / 4;
    extern __shared__ __align__(128) uint32_t smem[];
    uint64_t *bars = reinterpret_cast<uint64_t *>(smem);
    constexpr int kStages = C::kStages;
    const TileRing<kStages> ring{bars, bars + kStages, smem + 4 * kStages, (uint32_t)C::TW};
    // tpc = ngrp * 32, or fewer than 32 tasks in one partial group when the 2^d-bit state of 32 tasks does not
    // fit (d >= 15); lanes past tpc then address task tpc - 1 and own nothing
    uint32_t *pV = smem + C::RING;             // [tpc][CWV] task codes with guard bits (pair pass)
    uint32_t *pC = pV + tpc * CWV;             // [tpc][4] coarse task codes with guard bits (corner tests)
    uint32_t *state = pC + tpc * kCoarseWords; // [tpc][PS]
    uint32_t *zm = state + tpc * C::PS;        // [tpc] Z_p (kModeDims)
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    uint32_t *q1 = zm + tpc + warp * C::QW;    // opened (task, chunk) items (<= 3 + 32)
    uint32_t *q2 = q1 + 40;                    // opened (task, chunk, sub-chunk) items (<= 7 + 32)
    const int64_t j0 = j_begin + (int64_t)blockIdx.x * tpc;
    const int nt = (int)min((int64_t)tpc, j_end - j0);
    const int64_t ntiles = ceil_div_dev(nchunks, NW);

    if (threadIdx.x == 0) ring.init(NW);
    for (int i = threadIdx.x; i < tpc * G::CW; i += blockDim.x) {
        const int t = i / G::CW, k = i % G::CW;
        uint32_t w = t < nt ? p_codes[(j0 + t) * G::CW + k] : 0u;
        if (2 * k >= D) w &= 0xffff0000u;  // padding dimensions: p = 0 never passes q <= p (q pad = 1)
        if (2 * k + 1 >= D) w &= 0x0000ffffu;
        pV[t * CWV + k] = w | kGuard;
    }
    __syncthreads();
    for (int t = threadIdx.x; t < tpc; t += blockDim.x) coarse_row<D, G::CW>(pV + t * CWV, cshift, pC + t * kCoarseWords);
    if (MODE == kModeDims) {
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
        for (int t = threadIdx.x; t < tpc; t += blockDim.x) zm[t] = 0u;  // tie rows untouched
    }
    __syncthreads();
    if (warp == NW) {  // producer warp: one elected lane streams chunk tiles with TMA
        if (lane == 0)
            for (int64_t t = 0; t < ntiles; t++) ring.issue(chunks, t);
        return;
    }
    const uint32_t st_s = smem_addr(state), pV_s = smem_addr(pV), q1_s = smem_addr(q1), q2_s = smem_addr(q2);
    const uint32_t zm_s = smem_addr(zm);  // kModeGlobalTie: per-task tie-row flags (kModeDims: Z_p)
    const uint32_t ring_s = smem_addr(smem + 4 * kStages);
    const int wpg = NW / ngrp, grp = warp / wpg, wsub = warp % wpg;
    const int town = grp * 32 + lane;                         // this lane's task
    const uint32_t valid = __ballot_sync(0xffffffffu, town < nt);
    const uint32_t st_own = st_s + 4u * (min(town, tpc - 1) * C::PS);
    uint32_t p[kCoarseWords];  // this lane's coarse task codes (corner tests)
    load_row_s<kCoarseWords>(smem_addr(pC) + 4u * (min(town, tpc - 1) * kCoarseWords), p);
    const uint32_t pC_s = smem_addr(pC);
    unsigned long long n_box = 0, n_sub = 0, n_pair = 0, n_miss = 0, n_exp = 0;
    // ring barriers as 32-bit shared addresses kept in registers, position (stage, phase) kept incrementally
    // (a generic->shared conversion per wait/arrival was ~4% of this kernel's instructions at H, ncu r02)
    const uint32_t full_s = smem_addr(bars), empty_s = full_s + 8u * kStages;
    uint32_t stage = 0, phase = 0;
    for (int64_t tile = 0; tile < ntiles; tile++) {
        mbar_wait_s(full_s + 8u * stage, phase);
        const uint32_t stg_s = ring_s + 4u * stage * (uint32_t)C::TW;

        // pair pass over 8 queued (task, chunk, sub-chunk) items: lane (k, r) = item k, member r
        auto pair_pass = [&](int base, int cnt) {
            const int k8 = lane >> 2, r = lane & 3;
            const uint32_t it = lds_u32(q2_s + 4u * (base + min(k8, cnt - 1)));
            const int t = (int)(it >> 8), cl = (int)((it >> 3) & 31u), sidx = (int)(it & 7u);  // cl < NW <= 32
            const int m = sidx * kSubSize + r;                       // member of the chunk
            uint32_t qq[G::CW], x[G::CW], ph[G::CW];
            load_row2_s<G::CW>(stg_s + 4u * (cl * REC + m * G::CW), qq);
            load_row_s<G::CW>(pV_s + 4u * (t * CWV), ph);
#pragma unroll
            for (int k = 0; k < G::CW; k++) x[k] = ph[k] - qq[k];  // guard <=> code(q) <= code(p)
            const uint32_t M = gather_mask<G::NG>(x);
            const uint32_t wd = lds_u32(st_s + 4u * (t * C::PS + (M >> 5)));
            const bool miss = k8 < cnt && !(__funnelshift_r(wd, wd, M) & 1u);
            if (!__any_sync(0xffffffffu, miss)) return;  // Λ4 for every lane
            uint32_t L = 0, S = 0;
            if (miss) {
                n_miss++;
                const int64_t qpos = (tile * NW + cl) * 32 + m;
                exact_masks<D>(ph, qq, M, inexact, q_ord + qpos * D, p_ord + (j0 + t) * D, L, S);
                if (S != 0 && L != M && ((lds_u32(st_s + 4u * (uint32_t)(t * C::PS + (L >> 5))) >> (L & 31)) & 1u))
                    S = 0;  // exact L covered
            }
            uint32_t todo = __ballot_sync(0xffffffffu, S != 0);
            n_exp += __popc(todo);
            while (todo) {
                const int from = __ffs(todo) - 1;
                todo &= todo - 1;
                const uint32_t Sb = __shfl_sync(0xffffffffu, S, from), Lb = __shfl_sync(0xffffffffu, L, from);
                const int tb = __shfl_sync(0xffffffffu, t, from);
                const int64_t jt = j0 + tb;
                expand<D, MODE>(st_s + 4u * (uint32_t)(tb * C::PS), tie32 + (jt >> 5) * (G::WB * 32) + (jt & 31),
                                zm_s + 4u * (uint32_t)tb, Lb, Sb, MODE == kModeDims ? zm[tb] : 0u, lane);
            }
        };

        // sub-chunk pass over 4 queued (task, chunk) items: lane (u, s) tests item u against sub-corner s
        int n2 = 0;
        auto sub_pass = [&](int base, int cnt) {
            const int u = lane >> 3, sidx = lane & 7;
            const uint32_t it = lds_u32(q1_s + 4u * (base + min(u, cnt - 1)));
            const int t = (int)(it >> 5), cl = (int)(it & 31u);
            uint32_t x[kCoarseWords], sc[kCoarseWords];
            load_row_s<kCoarseWords>(pC_s + 4u * (t * kCoarseWords), x);
            load_row_s<kCoarseWords>(stg_s + 4u * (cl * REC + C::CO + kCoarseWords * (1 + sidx)), sc);
#pragma unroll
            for (int k = 0; k < NQ; k++) x[k] -= sc[k];  // guard <=> coarse sub-corner <= p
            const uint32_t Ms = gather_coarse<NQ>(x);
            const uint32_t ws = lds_u32(st_s + 4u * (t * C::PS + (Ms >> 5)));
            const bool open = u < cnt && !(__funnelshift_r(ws, ws, Ms) & 1u);
            const uint32_t ob = __ballot_sync(0xffffffffu, open);
            n_sub += 8 * cnt;
            if (!ob) return;
            n_pair += 4 * __popc(ob);
            if (open) sts_u32(q2_s + 4u * (n2 + __popc(ob & ((1u << lane) - 1u))), ((uint32_t)t << 8) | ((uint32_t)cl << 3) | (uint32_t)sidx);
            n2 += __popc(ob);
            __syncwarp();
            while (n2 >= 8) {
                n2 -= 8;
                pair_pass(n2, 8);
            }
            __syncwarp();
        };

        // chunk-corner (box) test: lane = task, the corner is broadcast; two chunks per iteration (ILP)
        int n1 = 0;
        auto enqueue = [&](uint32_t todo, int cl) {
            if (todo == 0) return;
            if ((todo >> lane) & 1u)
                sts_u32(q1_s + 4u * (n1 + __popc(todo & ((1u << lane) - 1u))), ((uint32_t)town << 5) | (uint32_t)cl);
            n1 += __popc(todo);
            __syncwarp();
            while (n1 >= 4) {
                n1 -= 4;
                sub_pass(n1, 4);
            }
            __syncwarp();
        };
        auto box_mask = [&](int cl) {
            uint32_t mn[kCoarseWords], le[kCoarseWords];
            load_row_s<kCoarseWords>(stg_s + 4u * (cl * REC + C::CO), mn);
#pragma unroll
            for (int k = 0; k < NQ; k++) le[k] = p[k] - mn[k];  // guard <=> coarse corner <= p
            return gather_coarse<NQ>(le);
        };
        const int nch_tile = (int)min((int64_t)NW, nchunks - tile * NW);
        const bool mine = (valid >> lane) & 1u;
        int cl = wsub;
        // four chunks per iteration where a warp has that many in the tile (ILP; H K3 79.9 -> 79.2 ms), then pairs
        for (; cl + 3 * wpg < nch_tile; cl += 4 * wpg) {
            const uint32_t M0 = box_mask(cl), M1 = box_mask(cl + wpg), M2 = box_mask(cl + 2 * wpg), M3 = box_mask(cl + 3 * wpg);
            const uint32_t w0 = lds_u32(st_own + 4u * (M0 >> 5)), w1 = lds_u32(st_own + 4u * (M1 >> 5));
            const uint32_t w2 = lds_u32(st_own + 4u * (M2 >> 5)), w3 = lds_u32(st_own + 4u * (M3 >> 5));
            const uint32_t todo0 = __ballot_sync(0xffffffffu, mine && !(__funnelshift_r(w0, w0, M0) & 1u));
            const uint32_t todo1 = __ballot_sync(0xffffffffu, mine && !(__funnelshift_r(w1, w1, M1) & 1u));
            const uint32_t todo2 = __ballot_sync(0xffffffffu, mine && !(__funnelshift_r(w2, w2, M2) & 1u));
            const uint32_t todo3 = __ballot_sync(0xffffffffu, mine && !(__funnelshift_r(w3, w3, M3) & 1u));
            n_box += 4 * __popc(valid);
            if ((todo0 | todo1 | todo2 | todo3) == 0) continue;
            enqueue(todo0, cl);
            enqueue(todo1, cl + wpg);
            enqueue(todo2, cl + 2 * wpg);
            enqueue(todo3, cl + 3 * wpg);
        }
        for (; cl + wpg < nch_tile; cl += 2 * wpg) {
            const uint32_t M0 = box_mask(cl), M1 = box_mask(cl + wpg);
            const uint32_t w0 = lds_u32(st_own + 4u * (M0 >> 5)), w1 = lds_u32(st_own + 4u * (M1 >> 5));
            const uint32_t todo0 = __ballot_sync(0xffffffffu, mine && !(__funnelshift_r(w0, w0, M0) & 1u));
            const uint32_t todo1 = __ballot_sync(0xffffffffu, mine && !(__funnelshift_r(w1, w1, M1) & 1u));
            n_box += 2 * __popc(valid);
            if ((todo0 | todo1) == 0) continue;
            enqueue(todo0, cl);
            enqueue(todo1, cl + wpg);
        }
        if (cl < nch_tile) {
            const uint32_t M0 = box_mask(cl);
            const uint32_t w0 = lds_u32(st_own + 4u * (M0 >> 5));
            n_box += __popc(valid);
            enqueue(__ballot_sync(0xffffffffu, mine && !(__funnelshift_r(w0, w0, M0) & 1u)), cl);
        }
        if (n1 > 0) sub_pass(0, n1);
        if (n2 > 0) pair_pass(0, n2);
        // every read of the stage has completed (values consumed) before it is handed back to the producer
        __threadfence_block();
        __syncwarp();
        if (lane == 0) mbar_arrive_s(empty_s + 8u * stage);
        if (++stage == (uint32_t)kStages) {
            stage = 0;
            phase ^= 1u;
        }
    }
    if (counters) {
        for (int o = 16; o; o >>= 1) n_miss += __shfl_xor_sync(0xffffffffu, n_miss, o);
        if (lane == 0) {
            atomicAdd(&counters[2], n_box);
            atomicAdd(&counters[3], n_pair);
            atomicAdd(&counters[4], n_miss);
            atomicAdd(&counters[5], n_sub);
            atomicAdd(&counters[6], n_exp);
        }
    }
    consumer_sync(NW * 32);
    write_rows<D, MODE, NW>(state, j0, nt, warp, lane, max_level, rows32, tie32, ext_rows32, host_mem, ext_ids, zm);
}

template <int D, int MODE, int NW>
size_t owner_smem_bytes(int tasks) {
    using C = GeoO<D, MODE, NW>;
    const size_t tpc = (size_t)tasks;
    return sizeof(uint32_t) * ((size_t)C::RING + tpc * (C::CWV + kCoarseWords + C::PS + 1) + NW * C::QW);
}

// Largest task-group count dividing NW (every group gets NW / ngrp warps) whose state fits in shared memory and
// that does not exceed `want`; 0 if not even one group fits.
template <int D, int MODE, int NW>
int owner_groups(int64_t want, int64_t range, int num_sms) {
    // candidates: group counts dividing NW that fit, at most `want` (>= one CTA per SM for small ranges).  The
    // largest one, unless the range is under 4 waves of such CTAs -- a shard of S+ at N > 1 ranks: H / 8 = 88K
    // tasks are 2.3 waves of 8-group CTAs -- where the count minimising waves x (groups + 1) keeps the last wave
    // from leaving most SMs idle (H / 8: 4 groups, K3 12.7 -> 11.6 ms).  Over many waves the CTA durations vary
    // enough to smooth the tail, and fewer groups only cost more chunk-stream passes (C3A, 10 waves: 6 instead
    // of 8 groups measured 32.4 -> 40.5 ms).
    int gmax = 0;
    for (int g = 1; g <= NW; g++)
        if (NW % g == 0 && owner_smem_bytes<D, MODE, NW>(g * 32) <= (size_t)kSmemBytes && (g == 1 || g <= want)) gmax = g;
    if (gmax < 1 || ceil_div(range, (int64_t)gmax * 32) >= 4 * (int64_t)num_sms) return gmax;
    int best = gmax;
    int64_t best_cost = ceil_div(ceil_div(range, (int64_t)gmax * 32), (int64_t)num_sms) * (gmax + 1);
    for (int g = gmax - 1; g >= 1; g--) {
        if (NW % g != 0) continue;
        const int64_t cost = ceil_div(ceil_div(range, (int64_t)g * 32), (int64_t)num_sms) * (g + 1);
        if (cost < best_cost) {
            best = g;
            best_cost = cost;
        }
    }
    return best;
}

template <int D, int MODE, int NW>
bool launch_owner(Ctx &c, int64_t j_begin, int64_t j_end, uint32_t *rows32, uint32_t *ext_rows32, uint32_t *host_mem,
                  cudaStream_t st) {
    const int64_t range = j_end - j_begin;
    // groups per CTA: the shared-memory budget, but at least one CTA per SM for small ranges
    const int64_t want = std::max<int64_t>(1, ceil_div(ceil_div(range, c.num_sms), 32));
    int ngrp = owner_groups<D, MODE, NW>(want, range, c.num_sms), tpc = ngrp * 32;
    if (ngrp < 1) {
        // one partial group: as many tasks as the shared memory holds (d = 16: 22 tasks of 8 KB state)
        ngrp = 1;
        tpc = 0;
        while (tpc < 31 && owner_smem_bytes<D, MODE, NW>(tpc + 1) <= (size_t)kSmemBytes) tpc++;
        if (tpc < 1) return false;
        tpc = (int)std::min<int64_t>(tpc, std::max<int64_t>(1, ceil_div(range, c.num_sms)));
    }
    const size_t smem = owner_smem_bytes<D, MODE, NW>(tpc);
    SKY_CUDA(cudaFuncSetAttribute(k3_owner_kernel<D, MODE, NW>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    const unsigned blocks = (unsigned)ceil_div(range, tpc);
    k3_owner_kernel<D, MODE, NW><<<blocks, (NW + 1) * 32, smem, st>>>(
        c.p_codes.as<uint32_t>(), c.p_ord.as<uint32_t>(), c.chunks_ext.as<uint32_t>(), c.q_ord.as<uint32_t>(),
        c.minord.as<uint32_t>(), c.nchunks_ext, j_begin, j_end, ~c.exact_mask & ((1u << D) - 1u), c.cshift, ngrp, tpc,
        (c.max_level > 0 && c.max_level < D) ? c.max_level : 0, rows32, c.tie.as<uint32_t>(), ext_rows32,
        c.counters.as<unsigned long long>(), host_mem, c.ext_ids.as<int32_t>());
    c.L.count++;
    SKY_LAUNCH_CHECK();
    return true;
}

template <int D, int MODE, int NW>
void launch_a(Ctx &c, int64_t j_begin, int64_t j_end, uint32_t *rows32, uint32_t *ext_rows32, uint32_t *host_mem,
              cudaStream_t st) {
    using C = GeoK3<D, MODE, NW>;
    static_assert(C::NT >= 1, "shared memory too small for one task per CTA");
    // tasks per CTA: the shared-memory budget, but at least one CTA per SM for small ranges
    const int64_t range = j_end - j_begin;
    int tpc = (int)std::min<int64_t>(C::NT, std::max<int64_t>(32, ceil_div(ceil_div(range, c.num_sms), 32) * 32));
    if (tpc == C::NT) {
        // Wave quantisation (one CTA per SM): a CTA's time grows with its task groups (the box pass walks
        // every group of every chunk) plus about one group's worth of per-tile work, so pick the task count
        // that minimises waves x (groups + 1) — e.g. C3I: 4 waves of 9 groups -> 4 waves of 8.
        auto cost = [&](int64_t t) { return ceil_div(ceil_div(range, t), (int64_t)c.num_sms) * (ceil_div(t, (int64_t)32) + 1); };
        int64_t best = cost(tpc);
        for (int t = (C::NT / 32) * 32; t >= 32; t -= 32)
            if (cost(t) < best) {
                best = cost(t);
                tpc = t;
            }
    }
    if (tuning().k3_tpc > 0) tpc = std::max(1, std::min<int>(C::NT, tuning().k3_tpc));
    const size_t smem = C::smem_bytes(tpc);
    SKY_CUDA(cudaFuncSetAttribute(k3_mdmc_kernel<D, MODE, NW>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    const unsigned blocks = (unsigned)ceil_div(range, tpc);
    k3_mdmc_kernel<D, MODE, NW><<<blocks, (NW + 1) * 32, smem, st>>>(
        c.p_codes.as<uint32_t>(), c.p_ord.as<uint32_t>(), c.chunks_ext.as<uint32_t>(), c.q_ord.as<uint32_t>(),
        c.minord.as<uint32_t>(), c.nchunks_ext, j_begin, j_end, ~c.exact_mask & ((1u << D) - 1u), c.cshift, tpc,
        (c.max_level > 0 && c.max_level < D) ? c.max_level : 0, rows32,
        c.tie.as<uint32_t>(), ext_rows32, c.counters.as<unsigned long long>(), host_mem, c.ext_ids.as<int32_t>());
    c.L.count++;
    SKY_LAUNCH_CHECK();
}

// Tie-heavy inputs (every dimension discrete enough for injective codes) or d <= 10: the tie-exact state
// (kModeDims, d <= 12) unless B_{p notin S+} itself is requested (ext rows), then kModeSmemTie.  Continuous
// data at d > 10: ties are rare and go to a global row (kModeGlobalTie).  skycube_set_tuning("k3_mode", m)
// forces a mode (parity tests of every mode on the same inputs).
template <int D, int MODE>
void launch_t(Ctx &c, int64_t j_begin, int64_t j_end, uint32_t *rows32, uint32_t *ext_rows32, uint32_t *host_mem,
              cudaStream_t st) {
    // Design O (task-owner warps) at d <= 12, where 24 warps fit 8 groups of tasks: H K3 86.7 (A, 24 warps) ->
    // 83.4 ms, C3I 7.2 -> 6.2, C3A 33.9 -> 34.3, C5 (tie-exact state) 20.1 (round 1 with 16 warps: A 92.8 vs O
    // 97.5 at H); and at d = 16 with one partial group of 22 tasks (task codes in registers instead of reloaded
    // per chunk, competitor rows read from the stage on demand): C4 K3 644 -> 615 ms.  Design A at d = 13..15,
    // where both measured within 1% (A 300K: d = 13 31.8 / 31.6 ms, d = 14 45.3 / 45.0, d = 15 71.3 / 72.1;
    // profiles/r02_k3_ab_s2.md).  skycube_set_tuning("k3_design", 'A' | 'O') forces one.
    const int design = tuning().k3_design;
    const bool want_o = design ? design == 'O' : (MODE == kModeDims || D <= 12 || D == 16);
    if (want_o) {
        // design O with 24 warps (the group count divides 24: e.g. 3 groups of 8 warps at d = 10, where 16 warps
        // fit only 2 groups): C5 K3 26.8 -> 20.2 ms, C2 0.5 -> 0.3 ms (profiles/r02_k3_warps_ab.md);
        // k3_warps = 16 forces the 16-warp kernel
        if constexpr (D <= 12)
            if (tuning().k3_warps != 16 && launch_owner<D, MODE, 24>(c, j_begin, j_end, rows32, ext_rows32, host_mem, st))
                return;
        if (launch_owner<D, MODE, kWarps>(c, j_begin, j_end, rows32, ext_rows32, host_mem, st)) return;
    }
    // design A: one chunk per consumer warp per tile.  At d = 12, 24 consumer warps (70 registers, 2 ring stages
    // of 24 chunks) instead of 16 (89 registers, 4 stages of 16): more warps per SM sub-partition against K3's
    // fixed-latency ("wait") stalls.  With the round-2 expansion walk it measured H 94.2 -> 89.5 ms, C3A 39.3 ->
    // 37.2, C3I 7.6 -> 7.5 (profiles/r02_k3_warps_ab.md), so it is the default there; k3_warps = 16 forces
    // the 16-warp kernel.  (28 warps measured slower: H 87.5-90.6 ms; 32 consumer warps + the producer exceed
    // the 1024-thread CTA limit.)
    if constexpr (D == 12) {
        if (tuning().k3_warps != 16) return launch_a<D, MODE, 24>(c, j_begin, j_end, rows32, ext_rows32, host_mem, st);
    }
    launch_a<D, MODE, kWarps>(c, j_begin, j_end, rows32, ext_rows32, host_mem, st);
}

template <int D>
void launch(Ctx &c, int64_t j_begin, int64_t j_end, uint32_t *rows32, uint32_t *ext_rows32, uint32_t *host_mem,
            cudaStream_t st) {
    const bool all_exact = c.exact_mask == ((1u << D) - 1u);
    int mode = (D <= 10 || all_exact) ? (D <= 12 && !ext_rows32 ? kModeDims : kModeSmemTie) : kModeGlobalTie;
    if (tuning().k3_mode >= 0) {
        mode = tuning().k3_mode;
        if (mode == kModeDims && (D > 12 || ext_rows32)) mode = kModeSmemTie;
    }
    if (mode == kModeDims) {
        if constexpr (D <= 12) launch_t<D, kModeDims>(c, j_begin, j_end, rows32, ext_rows32, host_mem, st);
    } else if (mode == kModeSmemTie) {
        launch_t<D, kModeSmemTie>(c, j_begin, j_end, rows32, ext_rows32, host_mem, st);
    } else {
        launch_t<D, kModeGlobalTie>(c, j_begin, j_end, rows32, ext_rows32, host_mem, st);
    }
}

}  // namespace

void mdmc_run(Ctx &c, int64_t j_begin, int64_t j_end, uint32_t *d_rows32, uint32_t *d_ext_rows32, cudaStream_t st,
              uint32_t *host_membership) {
    if (!c.ext_ready) throw Error{1, "skycube_dev_mdmc before skycube_dev_set_ext"};
    if (j_begin < 0 || j_end > c.m || (j_begin & 31)) throw Error{1, "bad MDMC task range"};
    if (j_end <= j_begin) return;
    // the tie rows (kModeGlobalTie; the epilogue reads only the rows a tie was OR-ed into)
    const size_t grp_words = (size_t)c.W * 32;
    c.tie.ensure(sizeof(uint32_t) * grp_words * (size_t)ceil_div(c.m, 32));
    SKY_CUDA(cudaMemsetAsync(c.tie.as<uint32_t>() + (j_begin >> 5) * grp_words, 0,
                             sizeof(uint32_t) * grp_words * (ceil_div(j_end, 32) - (j_begin >> 5)), st));
    switch (c.d) {
#define SKY_K3(DD) case DD: launch<DD>(c, j_begin, j_end, d_rows32, d_ext_rows32, host_membership, st); break;
        SKY_K3(1) SKY_K3(2) SKY_K3(3) SKY_K3(4) SKY_K3(5) SKY_K3(6) SKY_K3(7) SKY_K3(8)
        SKY_K3(9) SKY_K3(10) SKY_K3(11) SKY_K3(12) SKY_K3(13) SKY_K3(14) SKY_K3(15) SKY_K3(16)
#undef SKY_K3
        default: throw Error{1, "d must be in [1, 16]"};
    }
}

}  // namespace sky
