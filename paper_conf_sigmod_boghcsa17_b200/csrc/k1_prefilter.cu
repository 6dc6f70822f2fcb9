// k1_prefilter.cu — K1: the extended skyline S+(P) of Alg. 3 line 2 (L315).
//
//   p in S+(P)  <=>  no q in P strictly dominates p in the full space (Def. 1-2, delta = 2^d - 1).
//
// Competitors are all points in static-tree (Morton) order, in chunks of 32 with their lower corner
// (per-dimension minimum code).  q < p in every dimension requires code(q) <= code(p), hence
// corner < p in every dimension; a chunk whose corner fails that for a task cannot hold a dominator
// of it (the mask test of Eq. 1, applied to a whole leaf range of the static tree).
//
// CTA: kTasks tasks (consecutive tree positions) with their codes in shared memory, 16 consumer warps
// and one TMA producer warp streaming chunk tiles (16 chunk records per tile) through a 3-stage ring.
// Each consumer warp takes one chunk per tile: its 32 competitors sit in registers (one per lane);
//   box pass: lane l tests task tb+l against the chunk corner (SWAR strict compare, guard bits);
//   a ballot gives the tasks that need pair tests; for each, all lanes test their competitor
//   (codes strictly less in every dimension => dominated; equal codes in a non-injective dimension
//   fall back to the exact keys).  A dominated task is marked in a shared bit set and skipped after.
#include "ctx.cuh"
#include "tile_stream.cuh"

#include <algorithm>

namespace sky {
namespace {

constexpr int kWarps = kTileChunks;  // consumer warps = chunks per tile
constexpr int kTasks = 2048;       // tasks per CTA (<= 64 groups of 32)
constexpr int kStages = 3;

template <int CW>
__global__ void __launch_bounds__((kWarps + 1) * 32, 1) k1_prefilter_kernel(
    const uint32_t *__restrict__ chunks, const uint32_t *__restrict__ supers, const uint32_t *__restrict__ ord_sorted,
    int64_t n, int d, uint32_t inexact, int64_t nchunks, int64_t blk_offset, int64_t blk_step, int tpc,
    uint8_t *__restrict__ ext_sorted, unsigned long long *__restrict__ counters) {
    constexpr int CWP = CW | 1;         // odd row stride: conflict-free per-lane task loads
    constexpr int REC = 33 * CW;        // chunk record words
    constexpr int CWS = (CW + 3) & ~3;  // super-corner record words
    constexpr int TW = kTileChunks * REC + CWS;
    extern __shared__ __align__(128) uint32_t smem[];
    uint64_t *bars = reinterpret_cast<uint64_t *>(smem);
    const TileRing<kStages> ring{bars, bars + kStages, smem + 4 * kStages, (uint32_t)TW};
    uint32_t *pH = smem + 4 * kStages + kStages * TW;             // [tpc][CWP]
    uint32_t *domw = pH + tpc * CWP;                              // [tpc / 32] dominated bits
    uint32_t *needw = domw + tpc / 32;                            // [2][tpc / 32] tasks below the tile corner
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int64_t blk = blk_offset + (int64_t)blockIdx.x * blk_step;
    const int64_t s0 = blk * tpc;
    const int nt = (int)min((int64_t)tpc, n - s0);
    const int64_t ntiles = ceil_div_dev(nchunks, kTileChunks);

    if (threadIdx.x == 0) ring.init(kWarps);
    for (int i = threadIdx.x; i < tpc * CW; i += blockDim.x) {
        const int t = i / CW, k = i % CW;
        uint32_t w = t < nt ? chunks[((s0 + t) >> 5) * REC + ((s0 + t) & 31) * CW + k] : 0u;
        if (2 * k >= d) w |= 0x00007fffu;      // padding dimensions never reject
        if (2 * k + 1 >= d) w |= 0x7fff0000u;
        pH[t * CWP + k] = w | kGuard;
    }
    for (int i = threadIdx.x; i < tpc / 32; i += blockDim.x) {
        uint32_t dead = 0;  // tasks past n count as dominated
        for (int b = 0; b < 32; b++)
            if (i * 32 + b >= nt) dead |= 1u << b;
        domw[i] = dead;
    }
    __syncthreads();
    if (warp == kWarps) {
        if (lane == 0)
            for (int64_t t = 0; t < ntiles; t++) ring.issue2(chunks, kTileChunks * REC, supers, CWS, t);
        return;
    }
    // corner test: q < p needs code(q) < code(p) on injective dimensions but only code(q) <= code(p) on
    // the others (a bin may hold several values), so subtract 1 only in the injective lanes
    uint32_t csub[CW];
#pragma unroll
    for (int k = 0; k < CW; k++)
        csub[k] = (((inexact >> (2 * k)) & 1u) ? 0u : 1u) | (((inexact >> (2 * k + 1)) & 1u) ? 0u : 0x10000u);
    const int ngroups = (nt + 31) >> 5;
    unsigned long long n_box = 0, n_pair = 0;
    for (int64_t tile = 0; tile < ntiles; tile++) {
        ring.wait(tile);
        const uint32_t *stg = ring.stage(tile);
        uint32_t *need = needw + (tile & 1) * (tpc / 32);
        // phase A (super-chunk test, the upper level of the static tree): which live tasks lie strictly above
        // the tile's lower corner; groups of 32 tasks are spread over the warps
        {
            uint32_t sc[CW];
#pragma unroll
            for (int k = 0; k < CW; k++) sc[k] = stg[kTileChunks * REC + k] + csub[k];
            for (int g = warp; g < ngroups; g += kWarps) {
                const uint32_t dw = domw[g];
                uint32_t nb = 0;
                if (dw != 0xffffffffu) {
                    const int tt = g * 32 + lane;
                    uint32_t acc = 0xffffffffu;
#pragma unroll
                    for (int k = 0; k < CW; k++) acc &= pH[tt * CWP + k] - sc[k];
                    nb = __ballot_sync(0xffffffffu, !((dw >> lane) & 1u) && (acc & kGuard) == kGuard);
                    n_box += __popc(~dw);
                }
                if (lane == 0) need[g] = nb;
            }
        }
        consumer_sync(kWarps * 32);
        // phase B: one chunk per warp, only for the tasks of phase A
        const uint32_t *rec = stg + warp * REC;
        uint32_t q[CW], mn[CW];
#pragma unroll
        for (int k = 0; k < CW; k++) {
            q[k] = rec[lane * CW + k];
            mn[k] = rec[32 * CW + k] + csub[k];
        }
        __syncwarp();
        if (lane == 0) ring.release(tile);
        const int64_t c = tile * kTileChunks + warp;
        if (c >= nchunks) continue;
        const int64_t qpos = c * 32 + lane;
        // groups with work: lane l looks at groups l and l + 32 (ngroups <= kTasks / 32 = 64)
        uint64_t gm;
        {
            const uint32_t n0 = lane < ngroups ? need[lane] & ~domw[lane] : 0u;
            const uint32_t n1 = lane + 32 < ngroups ? need[lane + 32] & ~domw[lane + 32] : 0u;
            gm = (uint64_t)__ballot_sync(0xffffffffu, n0 != 0) | ((uint64_t)__ballot_sync(0xffffffffu, n1 != 0) << 32);
        }
        while (gm) {
            const int g = __ffsll((long long)gm) - 1;
            gm &= gm - 1;
            const uint32_t nw = need[g] & ~domw[g];
            if (nw == 0) continue;
            const int tt = g * 32 + lane;
            uint32_t acc = 0xffffffffu;
#pragma unroll
            for (int k = 0; k < CW; k++) acc &= pH[tt * CWP + k] - mn[k];  // chunk corner below p
            uint32_t todo = __ballot_sync(0xffffffffu, ((nw >> lane) & 1u) && (acc & kGuard) == kGuard);
            n_box += __popc(nw);
            n_pair += 32u * __popc(todo);
            while (todo) {
                const int b = __ffs(todo) - 1;
                todo &= todo - 1;
                const int ts = g * 32 + b;
                const uint32_t *ph = pH + ts * CWP;
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
                    const int64_t ps = s0 + ts;
#pragma unroll
                    for (int k = 0; k < CW; k++) {
#pragma unroll
                        for (int h = 0; h < 2; h++) {
                            const int i = 2 * k + h;
                            if (i >= d) continue;
                            const uint32_t qc = (q[k] >> (16 * h)) & 0xffffu, pc = (ph[k] >> (16 * h)) & 0x7fffu;
                            if (qc != pc) continue;
                            if (!((inexact >> i) & 1u) || !(ord_sorted[qpos * d + i] < ord_sorted[ps * d + i]))
                                dom = false;
                        }
                    }
                }
                if (__any_sync(0xffffffffu, dom) && lane == 0) atomicOr(&domw[ts >> 5], 1u << (ts & 31));
            }
        }
    }
    if (lane == 0 && counters) {
        atomicAdd(&counters[0], n_box);
        atomicAdd(&counters[1], n_pair);
    }
    consumer_sync(kWarps * 32);
    for (int t = threadIdx.x; t < nt; t += kWarps * 32) ext_sorted[s0 + t] = ((domw[t >> 5] >> (t & 31)) & 1u) ? 0 : 1;
}

template <int CW>
void launch(Ctx &c, int64_t blk_offset, int64_t blk_step, int64_t nblk_mine, int tpc, uint8_t *ext, cudaStream_t st) {
    constexpr int CWP = CW | 1;
    const size_t smem = sizeof(uint32_t) * (4 * kStages + (size_t)kStages * (kTileChunks * 33 * CW + ((CW + 3) & ~3)) +
                                            (size_t)tpc * CWP + 3 * (tpc / 32));
    SKY_CUDA(cudaFuncSetAttribute(k1_prefilter_kernel<CW>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    const uint32_t inexact = ~c.exact_mask & ((1u << c.d) - 1u);
    k1_prefilter_kernel<CW><<<(unsigned)nblk_mine, (kWarps + 1) * 32, smem, st>>>(
        c.chunks_all.as<uint32_t>(), c.supers_all.as<uint32_t>(), c.ord_sorted.as<uint32_t>(), c.n, c.d, inexact,
        c.nchunks_all, blk_offset, blk_step, tpc, ext, c.counters.as<unsigned long long>());
    c.L.count++;
    SKY_LAUNCH_CHECK();
}

}  // namespace

int prefilter_block_size(int64_t n, int64_t step);

// Blocks of tpc consecutive tree positions; block b is processed iff b % tile_step == tile_offset.
void prefilter_run(Ctx &c, int64_t tile_offset, int64_t tile_step, uint8_t *d_ext_sorted, cudaStream_t st) {
    if (!c.prepared) throw Error{1, "skycube_dev_prefilter before skycube_dev_prepare"};
    if (tile_step < 1 || tile_offset < 0) throw Error{1, "bad prefilter block range"};
    const int tpc = prefilter_block_size(c.n, tile_step);
    const int64_t nblk = ceil_div(c.n, tpc);
    if (tile_offset >= nblk) return;
    const int64_t mine = (nblk - 1 - tile_offset) / tile_step + 1;
    switch (c.dp / 2) {
        case 2: launch<2>(c, tile_offset, tile_step, mine, tpc, d_ext_sorted, st); break;
        case 4: launch<4>(c, tile_offset, tile_step, mine, tpc, d_ext_sorted, st); break;
        case 6: launch<6>(c, tile_offset, tile_step, mine, tpc, d_ext_sorted, st); break;
        case 8: launch<8>(c, tile_offset, tile_step, mine, tpc, d_ext_sorted, st); break;
        default: throw Error{1, "unsupported dimensionality"};
    }
}

// Tasks per CTA: up to kTasks, but small enough that every rank (step = number of ranks) gets at least
// two CTAs per SM.  Depends only on (n, step), so every rank derives the same blocks.
int prefilter_block_size(int64_t n, int64_t step) {
    const int64_t want = ceil_div(n, step * 2 * 148);
    return (int)std::max<int64_t>(32, std::min<int64_t>(kTasks, ceil_div(want, 32) * 32));
}

}  // namespace sky
