// k1_prefilter.cu — K1: the extended skyline S+(P) of Alg. 3 line 2 (L320).
//
//   p in S+(P)  <=>  no q in P strictly dominates p in the full space (Def. 1-2, delta = 2^d - 1).
//
// Competitors are all points in static-tree (Morton) order, in chunks of 32 with their lower corner
// (per-dimension minimum code), and tiles of 16 chunks with the tile's lower corner (the upper level of
// the static tree: 512 points).  q < p in every dimension requires code(q) <= code(p), hence corner < p in
// every dimension; a tile or chunk whose corner fails that for a task cannot hold a dominator of it (the
// mask test of Eq. 1, applied to a whole leaf range of the static tree).
//
// CTA: 16 consumer warps, each owning 32 consecutive tree positions (one task per lane, codes in
// registers), and one TMA producer warp streaming tiles through a ring; the warps never wait for each
// other (only for the ring).  The producer streams only the tiles that can hold a dominator of SOME task of
// the CTA -- tile corner < U in every dimension, U = the per-dimension maximum code of the CTA's 512 tasks
// (consecutive in Morton order, so U is a tight upper corner) -- and publishes each streamed tile's index
// with its ring slot, ending the stream with a sentinel.  Per streamed tile and warp:
//   tile test   every live lane tests the tile corner (SWAR strict compare with guard bits); if none
//               passes, the tile is done;
//   chunk test  for each of the 16 chunks, the lanes that passed test the chunk corner; a ballot gives the
//               tasks that need pair tests;
//   pair test   for each such task, every lane tests one competitor of the chunk (codes strictly less in
//               every dimension => dominated; equal codes in a non-injective dimension fall back to the
//               exact keys).  A dominated task leaves the warp's live mask.
#include <algorithm>

#include "ctx.cuh"
#include "tile_stream.cuh"

namespace sky {
namespace {

constexpr int kWarps = 16;                   // consumer warps (+1 producer warp)
constexpr int kTasks = kWarps * 32;          // tasks (tree positions) per CTA
// ring depth: 6 stages cover the bulk-copy latency of the (filtered) tile stream; at d > 12 (CW = 8) only 4
// fit with two CTAs per SM
template <int CW>
constexpr int stages_for() { return CW <= 6 ? 6 : 4; }

template <int CW>
__global__ void __launch_bounds__((kWarps + 1) * 32, 2) k1_prefilter_kernel(
    const uint32_t *__restrict__ chunks, const uint32_t *__restrict__ supers, const uint32_t *__restrict__ ord_sorted,
    int64_t n, int d, uint32_t inexact, int64_t nchunks, int64_t blk_offset, int64_t blk_step, int nsplit,
    uint8_t *__restrict__ ext_sorted, unsigned long long *__restrict__ counters) {
    constexpr int REC = 33 * CW;        // chunk record words: 32 code rows, then the lower corner
    constexpr int CWS = (CW + 3) & ~3;  // tile-corner record words
    constexpr int CWV = (CW + 3) & ~3;  // 16-byte task-code stride (broadcast vector loads)
    constexpr int TW = kTileChunks * REC + CWS;
    constexpr int kStages = stages_for<CW>();
    extern __shared__ __align__(128) uint32_t smem[];
    uint64_t *bars = reinterpret_cast<uint64_t *>(smem);
    const TileRing<kStages> ring{bars, bars + kStages, smem + 4 * kStages, (uint32_t)TW};
    uint32_t *pV = smem + 4 * kStages + kStages * TW;  // [kTasks][CWV] task codes with guard bits
    volatile int32_t *tile_idx = reinterpret_cast<volatile int32_t *>(pV + kTasks * CWV);  // [kStages]
    uint32_t *ucorner = pV + kTasks * CWV + kStages;   // [kWarps][CW] upper corner of each warp's tasks
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    // CTA = (block of kTasks tree positions, split of the competitor tiles): with nsplit > 1 the CTAs of a block
    // stream the tiles t = split (mod nsplit) each, and a task is outside S+ iff some split finds a dominator
    const int64_t blk = blk_offset + (int64_t)(blockIdx.x / nsplit) * blk_step;
    const int split = (int)(blockIdx.x % nsplit);
    const int64_t s0 = blk * kTasks;
    const int64_t ntiles = ceil_div_dev(nchunks, kTileChunks);

    if (threadIdx.x == 0) ring.init(kWarps);
    // corner test: q < p needs code(q) < code(p) on injective dimensions but only code(q) <= code(p) on
    // the others (a bin may hold several values), so subtract 1 only in the injective lanes:
    // corner < p  <=>  guard bits of (p - csub) - corner
    uint32_t csub[CW];
#pragma unroll
    for (int k = 0; k < CW; k++)
        csub[k] = (((inexact >> (2 * k)) & 1u) ? 0u : 1u) | (((inexact >> (2 * k + 1)) & 1u) ? 0u : 0x10000u);
    const int64_t ps = s0 + warp * 32 + lane;  // this lane's task (tree position)
    uint32_t p[CW], pm[CW];
    if (warp < kWarps) {
        const uint32_t *src = chunks + (ps >> 5) * REC + (ps & 31) * CW;  // code rows of the chunk records
#pragma unroll
        for (int k = 0; k < CW; k++) {
            uint32_t w = ps < n ? src[k] : 0u;
            if (2 * k >= d) w |= 0x00007fffu;  // padding dimensions never reject
            if (2 * k + 1 >= d) w |= 0x7fff0000u;
            p[k] = w | kGuard;
            pm[k] = p[k] - csub[k];
            pV[(warp * 32 + lane) * CWV + k] = p[k];
            uint32_t lo = ps < n ? (w & 0xffffu) : 0u, hi = ps < n ? (w >> 16) : 0u;
#pragma unroll
            for (int o = 16; o; o >>= 1) {
                lo = max(lo, __shfl_xor_sync(0xffffffffu, lo, o));
                hi = max(hi, __shfl_xor_sync(0xffffffffu, hi, o));
            }
            if (lane == 0) ucorner[warp * CW + k] = lo | (hi << 16);
        }
    }
    __syncthreads();
    if (warp == kWarps) {
        // producer warp: streams only the tiles whose corner is below the CTA's upper corner U (per-dimension
        // maximum code of its tasks) -- no other tile can hold a dominator of any task here -- and publishes
        // each streamed tile's index with its ring slot; -1 ends the stream.  The 32 lanes test 32 tile
        // corners at a time (independent loads); lane 0 issues the bulk copies in order.
        uint32_t um[CW];
#pragma unroll
        for (int k = 0; k < CW; k++) um[k] = 0;
#pragma unroll
        for (int w = 0; w < kWarps; w++) {
#pragma unroll
            for (int k = 0; k < CW; k++) {
                const uint32_t u = ucorner[w * CW + k];
                um[k] = max(um[k] & 0xffffu, u & 0xffffu) | (max(um[k] >> 16, u >> 16) << 16);
            }
        }
#pragma unroll
        for (int k = 0; k < CW; k++) um[k] = (um[k] | kGuard) - csub[k];
        int64_t slot = 0;
        for (int64_t t0 = 0; t0 < ntiles; t0 += 32) {
            const int64_t t = t0 + lane;
            bool pass = false;
            if (t < ntiles && (int)(t % nsplit) == split) {
                const uint32_t *sc = supers + t * CWS;
                uint32_t acc = 0xffffffffu;
#pragma unroll
                for (int k = 0; k < CW; k++) acc &= um[k] - __ldg(sc + k);
                pass = (acc & kGuard) == kGuard;
            }
            uint32_t m = __ballot_sync(0xffffffffu, pass);
            while (m) {
                const int b = __ffs(m) - 1;
                m &= m - 1;
                if (lane == 0) {
                    ring.wait_empty(slot);
                    tile_idx[slot % kStages] = (int32_t)(t0 + b);
                    ring.issue2_slot(chunks, kTileChunks * REC, supers, CWS, t0 + b, slot);
                }
                slot++;
            }
        }
        if (lane == 0) {
            ring.wait_empty(slot);
            tile_idx[slot % kStages] = -1;
            ring.arrive_full(slot);
        }
        return;
    }
    uint32_t live = __ballot_sync(0xffffffffu, ps < n);  // tasks not (yet) dominated
    unsigned long long n_box = 0, n_pair = 0;
    for (int64_t slot = 0;; slot++) {
        ring.wait(slot);
        const int64_t tile = tile_idx[slot % kStages];
        if (tile < 0) break;
        const uint32_t *stg = ring.stage(slot);
        uint32_t need = 0;
        if (live) {
            uint32_t acc = 0xffffffffu;
#pragma unroll
            for (int k = 0; k < CW; k++) acc &= pm[k] - stg[kTileChunks * REC + k];  // tile corner < p
            need = __ballot_sync(0xffffffffu, ((live >> lane) & 1u) && (acc & kGuard) == kGuard);
            n_box += __popc(live);
        }
        for (int ch = 0; need && ch < kTileChunks; ch++) {
            const int64_t c = tile * kTileChunks + ch;
            if (c >= nchunks) break;
            const uint32_t *rec = stg + ch * REC;
            uint32_t acc = 0xffffffffu;
#pragma unroll
            for (int k = 0; k < CW; k++) acc &= pm[k] - rec[32 * CW + k];  // chunk corner < p
            uint32_t todo = __ballot_sync(0xffffffffu, ((need >> lane) & 1u) && (acc & kGuard) == kGuard);
            n_box += __popc(need);
            if (!todo) continue;
            n_pair += 32u * __popc(todo);
            uint32_t q[CW];
#pragma unroll
            for (int k = 0; k < CW; k++) q[k] = rec[lane * CW + k];
            const int64_t qpos = c * 32 + lane;
            while (todo) {
                const int b = __ffs(todo) - 1;
                todo &= todo - 1;
                const uint32_t *ph = pV + (warp * 32 + b) * CWV;
                uint32_t lt = 0xffffffffu, le = 0xffffffffu;
#pragma unroll
                for (int k = 0; k < CW; k++) {
                    const uint32_t x = ph[k] - q[k];
                    le &= x;
                    lt &= x - 0x00010001u;
                }
                bool dom = (lt & kGuard) == kGuard;  // codes strictly smaller everywhere
                if (!dom && (le & kGuard) == kGuard && inexact) {
                    // equal codes somewhere: only non-injective dimensions may still be strictly less
                    dom = true;
                    const int64_t pp = s0 + warp * 32 + b;
#pragma unroll
                    for (int k = 0; k < CW; k++) {
#pragma unroll
                        for (int h = 0; h < 2; h++) {
                            const int i = 2 * k + h;
                            if (i >= d) continue;
                            const uint32_t qc = (q[k] >> (16 * h)) & 0xffffu, pc = (ph[k] >> (16 * h)) & 0x7fffu;
                            if (qc != pc) continue;
                            if (!((inexact >> i) & 1u) || !(ord_sorted[qpos * d + i] < ord_sorted[pp * d + i]))
                                dom = false;
                        }
                    }
                }
                if (__any_sync(0xffffffffu, dom)) {
                    live &= ~(1u << b);
                    need &= ~(1u << b);
                }
            }
        }
        // every read of the stage has completed before it is handed back to the producer
        __threadfence_block();
        __syncwarp();
        if (lane == 0) ring.release(slot);
    }
    if (lane == 0 && counters) {
        atomicAdd(&counters[0], n_box);
        atomicAdd(&counters[1], n_pair);
    }
    // nsplit == 1: the flag; else the block's flags were set to 1 before the launch and a split clears the tasks it
    // found dominated (plain byte stores of 0: idempotent across splits)
    if (ps < n && (nsplit == 1 || !((live >> lane) & 1u))) ext_sorted[ps] = (live >> lane) & 1u;
}

// ext[ps] = 1 for the tree positions of the blocks b = off (mod step) (the splits then clear the dominated ones)
__global__ void k1_fill_kernel(int64_t n, int64_t blk_offset, int64_t blk_step, int64_t nblk_mine, uint8_t *ext) {
    const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= nblk_mine * kTasks) return;
    const int64_t ps = (blk_offset + (i / kTasks) * blk_step) * kTasks + (i % kTasks);
    if (ps < n) ext[ps] = 1u;
}

template <int CW>
void launch(Ctx &c, int64_t blk_offset, int64_t blk_step, int64_t nblk_mine, uint8_t *ext, cudaStream_t st) {
    constexpr int kStages = stages_for<CW>();
    const size_t smem = sizeof(uint32_t) * (4 * kStages + (size_t)kStages * (kTileChunks * 33 * CW + ((CW + 3) & ~3)) +
                                            (size_t)kTasks * ((CW + 3) & ~3) + kStages + (size_t)kWarps * CW);
    SKY_CUDA(cudaFuncSetAttribute(k1_prefilter_kernel<CW>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    const uint32_t inexact = ~c.exact_mask & ((1u << c.d) - 1u);
    // Splits of the competitor stream when the rank's blocks fill fewer than 8 waves (two CTAs per SM): a rank's
    // K1 time is its slowest CTA, and at N = 8 ranks the 245 blocks of H are under one wave (K1 4.1 ms per rank
    // against 13.0 ms on one GPU); more, shorter CTAs spread it (a task's early exit then only covers its split).
    // Per-rank K1 at N = 8: H 4.1 -> 3.0 (4 waves) -> 2.7 ms (8 waves), C4 9.2 -> 5.8 -> 4.1 ms; one GPU unchanged.
    const int64_t slots = 2 * (int64_t)c.num_sms;
#ifndef SKY_K1_WAVES
#define SKY_K1_WAVES 8
#endif
    const int nsplit = (int)std::min<int64_t>(16, std::max<int64_t>(1, ceil_div(SKY_K1_WAVES * slots, nblk_mine)));
    if (nsplit > 1) {
        k1_fill_kernel<<<(unsigned)ceil_div(nblk_mine * kTasks, 256), 256, 0, st>>>(c.n, blk_offset, blk_step, nblk_mine,
                                                                               ext);
        c.L.count++;
        SKY_LAUNCH_CHECK();
    }
    k1_prefilter_kernel<CW><<<(unsigned)(nblk_mine * nsplit), (kWarps + 1) * 32, smem, st>>>(
        c.chunks_all.as<uint32_t>(), c.supers_all.as<uint32_t>(), c.ord_sorted.as<uint32_t>(), c.n, c.d, inexact,
        c.nchunks_all, blk_offset, blk_step, nsplit, ext, c.counters.as<unsigned long long>());
    c.L.count++;
    SKY_LAUNCH_CHECK();
}

}  // namespace

// Blocks of kTasks consecutive tree positions; block b is processed iff b % tile_step == tile_offset.
void prefilter_run(Ctx &c, int64_t tile_offset, int64_t tile_step, uint8_t *d_ext_sorted, cudaStream_t st) {
    if (!c.prepared) throw Error{1, "skycube_dev_prefilter before skycube_dev_prepare"};
    if (tile_step < 1 || tile_offset < 0) throw Error{1, "bad prefilter block range"};
    const int64_t nblk = ceil_div(c.n, kTasks);
    if (tile_offset >= nblk) return;
    const int64_t mine = (nblk - 1 - tile_offset) / tile_step + 1;
    switch (c.dp / 2) {
        case 2: launch<2>(c, tile_offset, tile_step, mine, d_ext_sorted, st); break;
        case 4: launch<4>(c, tile_offset, tile_step, mine, d_ext_sorted, st); break;
        case 6: launch<6>(c, tile_offset, tile_step, mine, d_ext_sorted, st); break;
        case 8: launch<8>(c, tile_offset, tile_step, mine, d_ext_sorted, st); break;
        default: throw Error{1, "unsupported dimensionality"};
    }
}

}  // namespace sky
