// prep.cu — K0 (validate + canonicalise + order-preserving keys), the key-sum order of Λ2, and
// K2 (per-dimension monotone 15-bit codes), plus the S+ gathers after the prefilter.
//
// Paper: Alg. 3 line 2 (L320) builds "quad tree T over S+(P)" with global pivots (median, quartiles,
// octiles: L338, L348-356; Fig. 3): every point gets, per dimension, its bin among
// statically defined global thresholds, and two points are compared through their bins (Eq. 1,
// L1312) before any exact dominance test.  This repo keeps that idea — global, monotone,
// per-dimension bins — but with 2^15 bins per dimension (dense ranks, made coarser only when a
// dimension has more than 2^15 distinct values), so that the bin comparison is exact for any
// dimension with <= 2^15 distinct values and almost always decisive otherwise.
//
// The leaves of the paper's static tree, in order, are reproduced by sorting the points on the Morton
// (bit-interleaved) key of their codes, top bits first: bit 1 of every dimension is the median split,
// bit 2 the quartile split, ... (L338 "median, then quartile, then octile").  Consecutive runs of 32
// points in that order are "chunks" whose per-dimension minimum codes bound every member; K1 and K3
// test a whole chunk against a task with one mask test (Eq. 1's idea, L1312) before any pair.
#include <algorithm>
#include <utility>

#include "ctx.cuh"

namespace sky {
namespace {

// Order-preserving image of a binary32 (after -0 -> +0): a < b  <=>  ord(a) < ord(b) for non-NaN.
__device__ __forceinline__ uint32_t ord_key(float x) {
    uint32_t b = __float_as_uint(x);
    if ((b & 0x7fffffffu) == 0) b = 0;             // -0 == +0 (reading Q11)
    return (b & 0x80000000u) ? ~b : (b | 0x80000000u);
}

// K0: one thread per point: order-preserving keys of every dimension, and the (dimension, key) sort items of the
// dimensions [db, de) (all of them on one GPU; a slice per rank in the multi-GPU prepare), local index i - db.
__global__ void k0_canon_kernel(const float *__restrict__ pts, int64_t n, int d, int db, int de,
                                uint32_t *__restrict__ ord, uint64_t *__restrict__ comp_keys,
                                uint32_t *__restrict__ comp_vals, uint32_t *__restrict__ nanflag) {
    const int64_t p = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (p >= n) return;
    bool nan = false;
    for (int i = 0; i < d; i++) {
        const float x = pts[p * d + i];
        nan |= (x != x);
        const uint32_t o = ord_key(x);
        ord[p * d + i] = o;
        if (i >= db && i < de) {
            comp_keys[(int64_t)(i - db) * n + p] = ((uint64_t)(i - db) << 32) | o;
            comp_vals[(int64_t)(i - db) * n + p] = (uint32_t)p;
        }
    }
    if (nan) atomicOr(nanflag, 1u);
}

// Morton key of the codes, rescaled to the full 15-bit range (exact dimensions have codes < R):
// bits_per_dim most significant bits of every dimension, interleaved, most significant level first.
__global__ void morton_kernel(const uint16_t *__restrict__ codes, const uint32_t *__restrict__ R, int64_t n, int d,
                              int dp, int bits_per_dim, uint64_t *__restrict__ keys, uint32_t *__restrict__ perm) {
    const int64_t p = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (p >= n) return;
    uint32_t sc[kMaxD];
    for (int i = 0; i < d; i++) {
        const uint32_t c = codes[p * dp + i], r = R[i];
        sc[i] = r <= kCodeLevels ? (uint32_t)(((uint64_t)c * kCodeLevels) / r) : c;
    }
    uint64_t key = 0;
    for (int b = 0; b < bits_per_dim; b++)
        for (int i = 0; i < d; i++) key = (key << 1) | ((sc[i] >> (14 - b)) & 1u);
    keys[p] = key;
    perm[p] = (uint32_t)p;
}

// Chunk records (kRecAll x cw words, K1): 32 consecutive points' code words, then the per-dimension minimum
// code words (the chunk's lower corner).  One warp per chunk.
__global__ void build_chunks_kernel(const uint32_t *__restrict__ codes, int64_t nchunks, int cw,
                                    uint32_t *__restrict__ chunks) {
    const int64_t c = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int lane = threadIdx.x & 31;
    if (c >= nchunks) return;
    uint32_t *rec = chunks + c * (int64_t)(kRecAll * cw);
    for (int k = 0; k < cw; k++) {
        const uint32_t w = codes[(c * 32 + lane) * cw + k];
        rec[lane * cw + k] = w;
        uint32_t lo = w & 0xffffu, hi = w >> 16;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            lo = min(lo, __shfl_xor_sync(0xffffffffu, lo, o));
            hi = min(hi, __shfl_xor_sync(0xffffffffu, hi, o));
        }
        if (lane == 0) rec[32 * cw + k] = lo | (hi << 16);
    }
}

// K3 chunk records (rec_ext_words(cw) words, ctx.cuh): the 32 members' code words, then the coarse lower
// corner of the chunk and of its 8 sub-chunks of kSubSize consecutive points (the level below), four 7-bit
// dimensions per word; padding dimensions (d..15) carry 127 (never below a task, whose padding is 0).  One warp
// per chunk; lane i of the coarse pass owns dimension i.
__global__ void build_chunks_ext_kernel(const uint32_t *__restrict__ codes, int64_t nchunks, int cw, int d,
                                        uint64_t cshift, uint32_t *__restrict__ chunks) {
    const int64_t c = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int lane = threadIdx.x & 31;
    if (c >= nchunks) return;
    uint32_t *rec = chunks + c * (int64_t)rec_ext_words(cw);
    uint32_t sub_lo[kCoarseRows], sub_hi[kCoarseRows];  // row 0: chunk corner, rows 1..8: sub-chunk corners
#pragma unroll
    for (int r = 0; r < kCoarseRows; r++) sub_lo[r] = 0x7fffu;
    for (int k = 0; k < cw; k++) {
        const uint32_t w = codes[(c * 32 + lane) * cw + k];
        rec[lane * cw + k] = w;
        uint32_t lo = w & 0xffffu, hi = w >> 16;
#pragma unroll
        for (int o = 1; o < kSubSize; o <<= 1) {
            lo = min(lo, __shfl_xor_sync(0xffffffffu, lo, o));
            hi = min(hi, __shfl_xor_sync(0xffffffffu, hi, o));
        }
        // lane s*kSubSize holds sub-chunk s's minimum; gather the 8 sub-corners and their minimum into every lane
        uint32_t clo = 0xffffu, chi = 0xffffu;
#pragma unroll
        for (int s = 0; s < 32 / kSubSize; s++) {
            const uint32_t a = __shfl_sync(0xffffffffu, lo, s * kSubSize), b = __shfl_sync(0xffffffffu, hi, s * kSubSize);
            if (lane == 2 * k) sub_lo[1 + s] = a;
            if (lane == 2 * k + 1) sub_lo[1 + s] = b;
            clo = min(clo, a);
            chi = min(chi, b);
        }
        if (lane == 2 * k) sub_lo[0] = clo;
        if (lane == 2 * k + 1) sub_lo[0] = chi;
    }
    // lane i < 16: the coarse corners of dimension i
    const uint32_t sh = (uint32_t)(cshift >> (4 * (lane & 15))) & 15u;
#pragma unroll
    for (int r = 0; r < kCoarseRows; r++) sub_hi[r] = lane < d ? min(sub_lo[r] >> sh, 127u) : 127u;
    // pack four dimensions per word: word g of row r = dims 4g..4g+3 (byte k = dim 4g+k)
#pragma unroll
    for (int r = 0; r < kCoarseRows; r++) {
        const uint32_t v = sub_hi[r];
        const uint32_t b1 = __shfl_down_sync(0xffffffffu, v, 1), b2 = __shfl_down_sync(0xffffffffu, v, 2),
                       b3 = __shfl_down_sync(0xffffffffu, v, 3);
        if (lane < 16 && (lane & 3) == 0)
            rec[32 * cw + r * kCoarseWords + (lane >> 2)] = v | (b1 << 8) | (b2 << 16) | (b3 << 24);
    }
}

// Super-chunk corners: per tile of kTileChunks chunk records, the per-dimension minimum of the chunk
// corners (the lower corner of 512 consecutive static-tree points).  One warp per tile.
__global__ void build_supers_kernel(const uint32_t *__restrict__ chunks, int64_t ntiles, int cw, int cws,
                                    uint32_t *__restrict__ supers) {
    const int64_t t = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int lane = threadIdx.x & 31;
    if (t >= ntiles) return;
    for (int k = 0; k < cws; k++) {
        uint32_t lo = 0x7fffu, hi = 0x7fffu;
        if (k < cw && lane < kTileChunks) {
            const uint32_t w = chunks[((t * kTileChunks + lane) * kRecAll + 32) * (int64_t)cw + k];
            lo = w & 0xffffu;
            hi = w >> 16;
        }
#pragma unroll
        for (int o = 16; o; o >>= 1) {
            lo = min(lo, __shfl_xor_sync(0xffffffffu, lo, o));
            hi = min(hi, __shfl_xor_sync(0xffffffffu, hi, o));
        }
        if (lane == 0) supers[t * cws + k] = lo | (hi << 16);
    }
}

// flags[t] = 1 iff t starts a run of equal (dim, key) in the per-dimension sorted order.
__global__ void k2_flags_kernel(const uint64_t *__restrict__ comp_keys, int64_t n, int64_t total,
                                uint32_t *__restrict__ flags) {
    const int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (t >= total) return;
    flags[t] = (t % n == 0 || comp_keys[t] != comp_keys[t - 1]) ? 1u : 0u;
}

// R[dim] = number of distinct values of dimension dim; minord[dim] = key of its minimum value.
__global__ void k2_distinct_kernel(const uint32_t *__restrict__ ex, const uint32_t *__restrict__ flags,
                                   const uint64_t *__restrict__ comp_keys, int64_t n, int d, uint32_t *__restrict__ R,
                                   uint32_t *__restrict__ minord) {
    const int i = threadIdx.x;
    if (i >= d) return;
    const int64_t a = (int64_t)i * n, b = (int64_t)(i + 1) * n - 1;
    R[i] = (ex[b] + flags[b]) - (ex[a] + flags[a]) + 1u;
    minord[i] = (uint32_t)comp_keys[a];
}

// code = dense rank if the dimension has <= 2^15 distinct values, else floor(rank * 2^15 / R):
// monotone in the value and equal for equal values (Λ3); injective iff R <= 2^15.
// codes of the slice's dimensions, dim-major: codes_dm[i][p] (i local); R indexed by local dimension
__global__ void k2_codes_kernel(const uint32_t *__restrict__ ex, const uint32_t *__restrict__ flags,
                                const uint32_t *__restrict__ comp_vals, const uint32_t *__restrict__ R,
                                int64_t n, int64_t total, uint16_t *__restrict__ codes_dm) {
    const int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (t >= total) return;
    const int dim = (int)(t / n);
    const int64_t a = (int64_t)dim * n;
    const uint32_t rank = (ex[t] + flags[t]) - (ex[a] + flags[a]);
    const uint32_t r = R[dim];
    const uint32_t code = r <= kCodeLevels ? rank : (uint32_t)(((uint64_t)rank * kCodeLevels) / r);
    codes_dm[(int64_t)dim * n + comp_vals[t]] = (uint16_t)code;
}

// codes_id[p][i] = codes_dm[i][p] for i < d; padding dimensions d..dp-1 carry code 1 on the competitor side
// (the task side zeroes them)
__global__ void k2_transpose_kernel(const uint16_t *__restrict__ codes_dm, int64_t n, int d, int dp,
                                    uint16_t *__restrict__ codes) {
    const int64_t p = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (p >= n) return;
    for (int i = 0; i < dp; i++) codes[p * dp + i] = i < d ? codes_dm[(int64_t)i * n + p] : (uint16_t)1;
}

__global__ void gather_sorted_kernel(const uint32_t *__restrict__ perm, const uint32_t *__restrict__ codes_id,
                                     const uint32_t *__restrict__ ord, int64_t n, int64_t npad, int d, int cw,
                                     uint32_t *__restrict__ codes_sorted, uint32_t *__restrict__ ord_sorted) {
    const int64_t s = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (s >= n) {  // padding up to whole chunk tiles: codes and exact keys that are never better than a task
        if (s < ((n + 31) / 32) * 32)
            for (int k = 0; k < cw; k++) codes_sorted[s * cw + k] = 0x7fff7fffu;
        // K1's tie path reads the exact keys of every competitor slot of a chunk it opens, padding included
        // (a task with code 0x7fff in every inexact dimension ties the padding codes there)
        if (s < npad)
            for (int i = 0; i < d; i++) ord_sorted[s * d + i] = 0xffffffffu;
        return;
    }
    const int64_t id = perm[s];
    for (int k = 0; k < cw; k++) codes_sorted[s * cw + k] = codes_id[id * cw + k];
    for (int i = 0; i < d; i++) ord_sorted[s * d + i] = ord[id * d + i];
}

__global__ void ext_scatter_kernel(const uint32_t *__restrict__ perm, const uint8_t *__restrict__ ext_sorted,
                                   int64_t n, uint32_t *__restrict__ ext_id_flag, uint32_t *__restrict__ key_flag) {
    const int64_t s = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (s >= n) return;
    const uint32_t f = ext_sorted[s] ? 1u : 0u;
    ext_id_flag[perm[s]] = f;
    key_flag[s] = f;
}

__global__ void ext_build_id_kernel(const uint32_t *__restrict__ ext_id_flag, const uint32_t *__restrict__ ext_idx,
                                    const uint32_t *__restrict__ codes_id, const uint32_t *__restrict__ ord,
                                    int64_t n, int d, int cw, int32_t *__restrict__ ext_ids,
                                    uint32_t *__restrict__ p_codes, uint32_t *__restrict__ p_ord) {
    const int64_t id = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (id >= n || !ext_id_flag[id]) return;
    const int64_t j = ext_idx[id];
    ext_ids[j] = (int32_t)id;
    for (int k = 0; k < cw; k++) p_codes[j * cw + k] = codes_id[id * cw + k];
    for (int i = 0; i < d; i++) p_ord[j * d + i] = ord[id * d + i];
}

__global__ void ext_build_key_kernel(const uint32_t *__restrict__ key_flag, const uint32_t *__restrict__ key_idx,
                                     const uint32_t *__restrict__ codes_sorted, const uint32_t *__restrict__ ord_sorted,
                                     int64_t n, int d, int cw, uint32_t *__restrict__ q_codes,
                                     uint32_t *__restrict__ q_ord) {
    const int64_t s = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (s >= n || !key_flag[s]) return;
    const int64_t jk = key_idx[s];
    for (int k = 0; k < cw; k++) q_codes[jk * cw + k] = codes_sorted[s * cw + k];
    for (int i = 0; i < d; i++) q_ord[jk * d + i] = ord_sorted[s * d + i];
}

inline unsigned blocks_for(int64_t n, int t) { return (unsigned)ceil_div(n > 0 ? n : 1, t); }

// key of a chunk = sum of its lower-corner codes (< 2^20 for d <= 16), the corner taken over the chunk's 32
// consecutive points of the code array
__global__ void chunk_key_kernel(const uint32_t *__restrict__ codes, int64_t nch, int cw, int d,
                                 uint64_t *__restrict__ keys, uint32_t *__restrict__ perm) {
    const int64_t ch = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (ch >= nch) return;
    uint64_t s = 0;
    for (int k = 0; k < cw; k++) {
        uint32_t lo = 0xffffu, hi = 0xffffu;
        for (int j = 0; j < 32; j++) {
            const uint32_t w = codes[(ch * 32 + j) * cw + k];
            lo = min(lo, w & 0xffffu);
            hi = min(hi, w >> 16);
        }
        if (2 * k < d) s += lo;
        if (2 * k + 1 < d) s += hi;
    }
    keys[ch] = s;
    perm[ch] = (uint32_t)ch;
}

// point j of new chunk c' <- point j of old chunk perm[c'] (codes and exact keys)
__global__ void permute_chunks_kernel(const uint32_t *__restrict__ perm, int64_t nch, int cw, int d,
                                      const uint32_t *__restrict__ codes, const uint32_t *__restrict__ ord,
                                      uint32_t *__restrict__ codes_out, uint32_t *__restrict__ ord_out) {
    const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= nch * 32) return;
    const int64_t src = (int64_t)perm[i >> 5] * 32 + (i & 31);
    for (int k = 0; k < cw; k++) codes_out[i * cw + k] = codes[src * cw + k];
    for (int k = 0; k < d; k++) ord_out[i * d + k] = ord[src * d + k];
}

__global__ void fill_kernel(uint32_t *a, int64_t from, int64_t to, uint32_t v) {
    const int64_t i = from + (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (i < to) a[i] = v;
}

// "never better" padding: codes 0x7fff in every lane, keys above every finite value
void pad_codes(uint32_t *codes, int64_t from, int64_t to, int cw, cudaStream_t st, Launches &L) {
    if (to <= from) return;
    fill_kernel<<<blocks_for((to - from) * cw, 256), 256, 0, st>>>(codes, from * cw, to * cw, 0x7fff7fffu);
    L.count++;
    SKY_LAUNCH_CHECK();
}

void pad_ord(uint32_t *ord, int64_t from, int64_t to, int d, cudaStream_t st, Launches &L) {
    if (to <= from) return;
    fill_kernel<<<blocks_for((to - from) * d, 256), 256, 0, st>>>(ord, from * d, to * d, 0xffffffffu);
    L.count++;
    SKY_LAUNCH_CHECK();
}

}  // namespace

// out[s] = OR over the k per-device flag vectors stage[g * n + s] (single-process multi-GPU prefilter)
__global__ void or_flags_kernel(const uint8_t *__restrict__ stage, int k, int64_t n, uint8_t *__restrict__ out) {
    const int64_t s = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (s >= n) return;
    uint8_t v = 0;
    for (int g = 0; g < k; g++) v |= stage[(int64_t)g * n + s];
    out[s] = v;
}

void or_flags(Ctx &c, const uint8_t *stage, int k, int64_t n, uint8_t *out, cudaStream_t st) {
    or_flags_kernel<<<blocks_for(n, 256), 256, 0, st>>>(stage, k, n, out);
    c.L.count++;
    SKY_LAUNCH_CHECK();
}

// K0 + K2 on the dimensions [db, de): order-preserving keys of every dimension (c.ord), and for the slice the
// dense-rank codes (dim-major, codes_dm[i - db][p]), distinct-value counts R[i] and minimum keys minord[i]
// (arrays indexed by global dimension; only the slice's entries are written).  One GPU: the whole range.
void prep_dims(Ctx &c, const float *d_points, int64_t n, int d, int db, int de, uint16_t *codes_dm, uint32_t *R,
               uint32_t *minord, cudaStream_t st) {
    c.n = n;
    c.d = d;
    c.dp = dpad_of(d);
    c.W = words_per_row(d);
    c.prepared = false;
    c.ext_ready = false;
    c.m = 0;
    const int nl = de - db;
    const int64_t nd = n * (nl > 0 ? nl : 1);
    c.ord.ensure(sizeof(uint32_t) * n * d);
    c.comp_keys.ensure(sizeof(uint64_t) * nd);
    c.comp_vals.ensure(sizeof(uint32_t) * nd);
    c.keys_alt.ensure(sizeof(uint64_t) * std::max<int64_t>(nd, n));
    c.vals_alt.ensure(sizeof(uint32_t) * std::max<int64_t>(nd, n));
    const int64_t cnt = std::max<int64_t>(radix_scratch_counts(nd), radix_scratch_counts(n));
    c.counts.ensure(sizeof(uint32_t) * cnt);
    c.scan_tmp.ensure(scan_tmp_bytes(std::max<int64_t>(cnt, nd)));
    c.flags.ensure(sizeof(uint32_t) * nd);
    c.scanned.ensure(sizeof(uint32_t) * nd);
    c.nanflag.ensure(sizeof(uint32_t));

    SKY_CUDA(cudaMemsetAsync(c.nanflag.p, 0, sizeof(uint32_t), st));
    k0_canon_kernel<<<blocks_for(n, 256), 256, 0, st>>>(d_points, n, d, db, de, c.ord.as<uint32_t>(),
                                                        c.comp_keys.as<uint64_t>(), c.comp_vals.as<uint32_t>(),
                                                        c.nanflag.as<uint32_t>());
    c.L.count++;
    SKY_LAUNCH_CHECK();
    uint32_t nan = 0;
    SKY_CUDA(cudaMemcpyAsync(&nan, c.nanflag.p, sizeof(uint32_t), cudaMemcpyDeviceToHost, st));
    SKY_CUDA(cudaStreamSynchronize(st));
    if (nan) throw Error{2, "NaN in input points"};
    if (nl <= 0) return;

    // K2: per-dimension sort of (dim, key) -> dense ranks -> codes.
    int dbits = 0;
    while ((1 << dbits) < nl) dbits++;
    radix_sort_u64(c.comp_keys.as<uint64_t>(), c.comp_vals.as<uint32_t>(), nd, 32 + dbits, c.keys_alt.as<uint64_t>(),
                   c.vals_alt.as<uint32_t>(), c.counts.as<uint32_t>(), c.scan_tmp.p, st, c.L);
    k2_flags_kernel<<<blocks_for(nd, 256), 256, 0, st>>>(c.comp_keys.as<uint64_t>(), n, nd, c.flags.as<uint32_t>());
    c.L.count++;
    SKY_LAUNCH_CHECK();
    exclusive_scan_u32(c.flags.as<uint32_t>(), c.scanned.as<uint32_t>(), nd, c.scan_tmp.p, st, c.L);
    k2_distinct_kernel<<<1, 32, 0, st>>>(c.scanned.as<uint32_t>(), c.flags.as<uint32_t>(), c.comp_keys.as<uint64_t>(), n,
                                         nl, R + db, minord + db);
    c.L.count++;
    SKY_LAUNCH_CHECK();
    k2_codes_kernel<<<blocks_for(nd, 256), 256, 0, st>>>(c.scanned.as<uint32_t>(), c.flags.as<uint32_t>(),
                                                         c.comp_vals.as<uint32_t>(), R + db, n, nd, codes_dm);
    c.L.count++;
    SKY_LAUNCH_CHECK();
}

// The rest of the preparation from every dimension's codes (dim-major codes_dm[d][n], R[d], minord[d], device):
// codes by id, the static-tree (Morton) order, chunk records and tile corners (K1 competitors).
void prep_finish(Ctx &c, const uint16_t *codes_dm, const uint32_t *R, const uint32_t *minord, cudaStream_t st) {
    const int64_t n = c.n;
    const int d = c.d;
    const int cw = c.dp / 2;  // 32-bit code words per point
    const int64_t npad = ceil_div(n, 32) * 32 + kChunkTilePad;  // whole chunks + whole chunk tiles
    c.keysum.ensure(sizeof(uint64_t) * n);
    c.perm.ensure(sizeof(uint32_t) * n);
    c.keys_alt.ensure(sizeof(uint64_t) * n);
    c.vals_alt.ensure(sizeof(uint32_t) * n);
    c.counts.ensure(sizeof(uint32_t) * radix_scratch_counts(n));
    c.scan_tmp.ensure(scan_tmp_bytes(std::max<int64_t>(radix_scratch_counts(n), n)));
    c.rbuf.ensure(sizeof(uint32_t) * kMaxD);
    c.minord.ensure(sizeof(uint32_t) * kMaxD);
    c.codes_id.ensure(sizeof(uint16_t) * n * c.dp);
    c.codes_sorted.ensure(sizeof(uint16_t) * npad * c.dp);
    c.ord_sorted.ensure(sizeof(uint32_t) * npad * d);
    c.chunks_all.ensure(sizeof(uint32_t) * (npad / 32) * kRecAll * cw);
    if (R != c.rbuf.as<uint32_t>())
        SKY_CUDA(cudaMemcpyAsync(c.rbuf.p, R, sizeof(uint32_t) * d, cudaMemcpyDeviceToDevice, st));
    if (minord != c.minord.as<uint32_t>())
        SKY_CUDA(cudaMemcpyAsync(c.minord.p, minord, sizeof(uint32_t) * d, cudaMemcpyDeviceToDevice, st));
    k2_transpose_kernel<<<blocks_for(n, 256), 256, 0, st>>>(codes_dm, n, d, c.dp, c.codes_id.as<uint16_t>());
    c.L.count++;
    SKY_LAUNCH_CHECK();
    SKY_CUDA(cudaMemcpyAsync(c.R, c.rbuf.p, sizeof(uint32_t) * d, cudaMemcpyDeviceToHost, st));
    // static-tree leaf order: Morton key of the codes (top bits first), then chunks of 32
    // (at most 32 key bits: the top bits decide the chunks of 32 and their sub-chunks -- 2^15 chunks at n = 1M --
    // and the stable sort keeps id order below; 32 bits sort in 4 radix passes instead of 8)
    const int bits_per_dim = std::min(15, 32 / d);
    morton_kernel<<<blocks_for(n, 256), 256, 0, st>>>(c.codes_id.as<uint16_t>(), c.rbuf.as<uint32_t>(), n, d, c.dp,
                                                      bits_per_dim, c.keysum.as<uint64_t>(), c.perm.as<uint32_t>());
    c.L.count++;
    SKY_LAUNCH_CHECK();
    radix_sort_u64(c.keysum.as<uint64_t>(), c.perm.as<uint32_t>(), n, bits_per_dim * d, c.keys_alt.as<uint64_t>(),
                   c.vals_alt.as<uint32_t>(), c.counts.as<uint32_t>(), c.scan_tmp.p, st, c.L);
    gather_sorted_kernel<<<blocks_for(npad, 256), 256, 0, st>>>(c.perm.as<uint32_t>(), c.codes_id.as<uint32_t>(),
                                                               c.ord.as<uint32_t>(), n, npad, d, cw,
                                                               c.codes_sorted.as<uint32_t>(), c.ord_sorted.as<uint32_t>());
    c.L.count++;
    SKY_LAUNCH_CHECK();
    const int64_t nch = ceil_div(n, 32);
    pad_codes(c.codes_sorted.as<uint32_t>(), nch * 32, npad, cw, st, c.L);
    build_chunks_kernel<<<blocks_for((npad / 32) * 32, 256), 256, 0, st>>>(c.codes_sorted.as<uint32_t>(), npad / 32, cw,
                                                                          c.chunks_all.as<uint32_t>());
    c.L.count++;
    SKY_LAUNCH_CHECK();
    c.nchunks_all = nch;
    const int64_t ntiles = ceil_div(nch, kTileChunks);
    c.supers_all.ensure(sizeof(uint32_t) * ntiles * super_words(cw));
    build_supers_kernel<<<blocks_for(ntiles * 32, 256), 256, 0, st>>>(c.chunks_all.as<uint32_t>(), ntiles, cw,
                                                                      super_words(cw), c.supers_all.as<uint32_t>());
    c.L.count++;
    SKY_LAUNCH_CHECK();
    SKY_CUDA(cudaStreamSynchronize(st));
    c.exact_mask = 0;
    c.cshift = 0;
    for (int i = 0; i < d; i++) {
        if (c.R[i] <= kCodeLevels) c.exact_mask |= 1u << i;
        // coarse-code shift: the codes of dimension i lie in [0, min(R_i, 2^15)); shift them into 7 bits
        const uint32_t top = std::min<uint32_t>(c.R[i], kCodeLevels) - 1u;
        int sh = 0;
        while ((top >> sh) > 127u) sh++;
        c.cshift |= (uint64_t)sh << (4 * i);
    }
    c.prepared = true;
}

void prep_run(Ctx &c, const float *d_points, int64_t n, int d, cudaStream_t st) {
    c.codes_dm.ensure(sizeof(uint16_t) * n * d);
    c.rbuf.ensure(sizeof(uint32_t) * kMaxD);
    c.minord.ensure(sizeof(uint32_t) * kMaxD);
    prep_dims(c, d_points, n, d, 0, d, c.codes_dm.as<uint16_t>(), c.rbuf.as<uint32_t>(), c.minord.as<uint32_t>(), st);
    prep_finish(c, c.codes_dm.as<uint16_t>(), c.rbuf.as<uint32_t>(), c.minord.as<uint32_t>(), st);
}

void ext_build(Ctx &c, const uint8_t *d_ext_sorted, cudaStream_t st) {
    if (!c.prepared) throw Error{1, "skycube_dev_set_ext before skycube_dev_prepare"};
    const int64_t n = c.n;
    const int d = c.d;
    const int cw = c.dp / 2;
    c.ext_id_flag.ensure(sizeof(uint32_t) * n);
    c.ext_idx.ensure(sizeof(uint32_t) * n);
    c.key_flag.ensure(sizeof(uint32_t) * n);
    c.key_idx.ensure(sizeof(uint32_t) * n);
    c.scan_tmp.ensure(scan_tmp_bytes(n));
    ext_scatter_kernel<<<blocks_for(n, 256), 256, 0, st>>>(c.perm.as<uint32_t>(), d_ext_sorted, n,
                                                           c.ext_id_flag.as<uint32_t>(), c.key_flag.as<uint32_t>());
    c.L.count++;
    SKY_LAUNCH_CHECK();
    exclusive_scan_u32(c.ext_id_flag.as<uint32_t>(), c.ext_idx.as<uint32_t>(), n, c.scan_tmp.p, st, c.L);
    exclusive_scan_u32(c.key_flag.as<uint32_t>(), c.key_idx.as<uint32_t>(), n, c.scan_tmp.p, st, c.L);
    uint32_t last[2];
    SKY_CUDA(cudaMemcpyAsync(&last[0], c.ext_idx.as<uint32_t>() + (n - 1), sizeof(uint32_t), cudaMemcpyDeviceToHost, st));
    SKY_CUDA(cudaMemcpyAsync(&last[1], c.ext_id_flag.as<uint32_t>() + (n - 1), sizeof(uint32_t), cudaMemcpyDeviceToHost, st));
    SKY_CUDA(cudaStreamSynchronize(st));
    const int64_t m = (int64_t)last[0] + last[1];
    c.m = m;
    const int64_t mm = m > 0 ? m : 1;
    const int64_t mpad = ceil_div(mm, kQPad) * kQPad;  // whole tiles of every K3 design
    c.ext_ids.ensure(sizeof(int32_t) * mm);
    c.p_codes.ensure(sizeof(uint16_t) * (mm + 32) * c.dp);
    c.p_ord.ensure(sizeof(uint32_t) * mm * d);
    c.q_codes.ensure(sizeof(uint16_t) * mpad * c.dp);
    c.q_ord.ensure(sizeof(uint32_t) * mpad * d);
    c.chunks_ext.ensure(sizeof(uint32_t) * (mpad / 32) * rec_ext_words(cw));
    ext_build_id_kernel<<<blocks_for(n, 256), 256, 0, st>>>(c.ext_id_flag.as<uint32_t>(), c.ext_idx.as<uint32_t>(),
                                                            c.codes_id.as<uint32_t>(), c.ord.as<uint32_t>(), n, d, cw,
                                                            c.ext_ids.as<int32_t>(), c.p_codes.as<uint32_t>(),
                                                            c.p_ord.as<uint32_t>());
    c.L.count++;
    SKY_LAUNCH_CHECK();
    // competitor stream: S+ in static-tree (Morton) order, padded with never-better points
    ext_build_key_kernel<<<blocks_for(n, 256), 256, 0, st>>>(c.key_flag.as<uint32_t>(), c.key_idx.as<uint32_t>(),
                                                             c.codes_sorted.as<uint32_t>(), c.ord_sorted.as<uint32_t>(),
                                                             n, d, cw, c.q_codes.as<uint32_t>(), c.q_ord.as<uint32_t>());
    c.L.count++;
    SKY_LAUNCH_CHECK();
    pad_codes(c.q_codes.as<uint32_t>(), m, mpad, cw, st, c.L);
    pad_ord(c.q_ord.as<uint32_t>(), m, mpad, d, st, c.L);
    // Chunks of the static-tree order, then visited strongest lower corner first (smallest sum of corner
    // codes): B_{p notin S+} saturates early, so later chunks resolve by their corner test.
    const int64_t nch = ceil_div(m, 32);
    c.chunk_keys.ensure(sizeof(uint64_t) * nch);
    c.chunk_perm.ensure(sizeof(uint32_t) * nch);
    c.q_codes_alt.ensure(sizeof(uint32_t) * mpad * cw);
    c.q_ord_alt.ensure(sizeof(uint32_t) * mpad * d);
    chunk_key_kernel<<<blocks_for(nch, 256), 256, 0, st>>>(c.q_codes.as<uint32_t>(), nch, cw, d,
                                                           c.chunk_keys.as<uint64_t>(), c.chunk_perm.as<uint32_t>());
    c.L.count++;
    SKY_LAUNCH_CHECK();
    radix_sort_u64(c.chunk_keys.as<uint64_t>(), c.chunk_perm.as<uint32_t>(), nch, 20, c.keys_alt.as<uint64_t>(),
                   c.vals_alt.as<uint32_t>(), c.counts.as<uint32_t>(), c.scan_tmp.p, st, c.L);
    permute_chunks_kernel<<<blocks_for(nch * 32, 256), 256, 0, st>>>(c.chunk_perm.as<uint32_t>(), nch, cw, d,
                                                                     c.q_codes.as<uint32_t>(), c.q_ord.as<uint32_t>(),
                                                                     c.q_codes_alt.as<uint32_t>(),
                                                                     c.q_ord_alt.as<uint32_t>());
    c.L.count++;
    SKY_LAUNCH_CHECK();
    std::swap(c.q_codes, c.q_codes_alt);
    std::swap(c.q_ord, c.q_ord_alt);
    pad_codes(c.q_codes.as<uint32_t>(), nch * 32, mpad, cw, st, c.L);
    pad_ord(c.q_ord.as<uint32_t>(), nch * 32, mpad, d, st, c.L);
    build_chunks_ext_kernel<<<blocks_for(mpad, 256), 256, 0, st>>>(c.q_codes.as<uint32_t>(), mpad / 32, cw, d, c.cshift,
                                                                  c.chunks_ext.as<uint32_t>());
    c.L.count++;
    SKY_LAUNCH_CHECK();
    c.nchunks_ext = nch;
    c.ext_ready = true;
}

}  // namespace sky
