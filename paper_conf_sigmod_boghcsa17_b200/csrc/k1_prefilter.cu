// k1_prefilter.cu — K1: the extended skyline S+(P) of Alg. 3 line 2 (L315).
//
//   p in S+(P)  <=>  no q in P strictly dominates p in the full space (Def. 1-2, delta = 2^d - 1).
//
// Λ2: key(x) = sum_i ord(x[i]) is exact in 64 bits and q strictly dominates p implies
// key(q) < key(p).  Points are sorted by key (prep.cu), so a point at sorted position s only needs
// the positions t < s as candidates; scanning them from the smallest key first finds the strong
// dominators early, and a block stops as soon as every one of its points is dominated.
//
// Each candidate is first rejected through the 15-bit codes: q < p in every dimension requires
// code(q) <= code(p) in every dimension (Λ3), which is a SWAR test of 16-bit lanes with a guard bit
// (two dimensions per 32-bit word; no branches).  Survivors get the exact test on the
// order-preserving keys.
#include "ctx.cuh"
#include "tile_stream.cuh"

namespace sky {
namespace {

constexpr int kThreads = kPrefilterTile;  // one sorted position per thread
constexpr int kTQ = 256;                  // candidates per shared-memory tile
constexpr int kU = 4;                     // candidates per inner iteration

template <int CW>
__global__ void __launch_bounds__(kThreads) k1_prefilter_kernel(
    const uint32_t *__restrict__ codes_sorted, const uint32_t *__restrict__ ord_sorted, int64_t n, int d,
    int64_t tile_offset, int64_t tile_step, int64_t ntiles_mine, uint8_t *__restrict__ ext_sorted) {
    extern __shared__ __align__(128) uint32_t smem[];
    const TileStream2 ts{reinterpret_cast<uint64_t *>(smem), smem + 4, (uint32_t)(kTQ * CW)};
    const int64_t tile = tile_offset + (ntiles_mine - 1 - (int64_t)blockIdx.x) * tile_step;  // heaviest first
    const int64_t s = tile * kThreads + threadIdx.x;
    const bool valid = s < n;
    if (threadIdx.x == 0) ts.init();
    uint32_t pH[CW];
#pragma unroll
    for (int k = 0; k < CW; k++) {
        uint32_t w = valid ? codes_sorted[s * CW + k] : 0u;
        // padding halves (dimensions >= d) must never reject: make p maximal there
        if (2 * k >= d) w |= 0x00007fffu;
        if (2 * k + 1 >= d) w |= 0x7fff0000u;
        pH[k] = w | kGuard;
    }
    const int64_t s_hi = min(n, (tile + 1) * (int64_t)kThreads);
    const int64_t nqt = ceil_div_dev(s_hi, kTQ);
    __syncthreads();
    int64_t issued = 0;
    if (threadIdx.x == 0) {
        ts.issue(codes_sorted, 0);
        if (nqt > 1) ts.issue(codes_sorted, 1);
    }
    issued = nqt > 1 ? 2 : 1;
    bool dom = !valid;
    int64_t qt = 0;
    for (; qt < nqt; qt++) {
        ts.wait(qt);
        const uint32_t *qs = ts.stage(qt);
        if (!dom) {
#pragma unroll 1
            for (int t = 0; t < kTQ; t += kU) {
                uint32_t cand = 0;
#pragma unroll
                for (int u = 0; u < kU; u++) {
                    uint32_t acc = 0xffffffffu;
#pragma unroll
                    for (int k = 0; k < CW; k++) acc &= pH[k] - qs[(t + u) * CW + k];  // guard <=> code(q) <= code(p)
                    cand |= ((acc & kGuard) == kGuard) ? (1u << u) : 0u;
                }
                if (cand == 0) continue;
#pragma unroll
                for (int u = 0; u < kU; u++) {
                    const int64_t q = qt * kTQ + t + u;
                    if (((cand >> u) & 1u) && q < s && !dom) {
                        bool strict = true;
                        for (int i = 0; i < d && strict; i++) strict = ord_sorted[q * d + i] < ord_sorted[s * d + i];
                        dom = strict;
                    }
                }
                if (dom) break;
            }
        }
        const int all = __syncthreads_and(dom);
        if (all) break;
        if (threadIdx.x == 0 && qt + 2 < nqt) ts.issue(codes_sorted, qt + 2);
        issued = min(nqt, qt + 3);
    }
    // drain bulk copies still in flight before the CTA's shared memory is released
    if (threadIdx.x == 0)
        for (int64_t t = qt + 1; t < issued; t++) ts.wait(t);
    if (valid) ext_sorted[s] = dom ? 0 : 1;
}

template <int CW>
void launch(Ctx &c, int64_t tile_offset, int64_t tile_step, int64_t ntiles_mine, uint8_t *ext, cudaStream_t st) {
    const size_t smem = sizeof(uint32_t) * (4 + 2 * (size_t)kTQ * CW);
    k1_prefilter_kernel<CW><<<(unsigned)ntiles_mine, kThreads, smem, st>>>(
        c.codes_sorted.as<uint32_t>(), c.ord_sorted.as<uint32_t>(), c.n, c.d, tile_offset, tile_step, ntiles_mine, ext);
    c.L.count++;
    SKY_LAUNCH_CHECK();
}

}  // namespace

void prefilter_run(Ctx &c, int64_t tile_offset, int64_t tile_step, uint8_t *d_ext_sorted, cudaStream_t st) {
    if (!c.prepared) throw Error{1, "skycube_dev_prefilter before skycube_dev_prepare"};
    if (tile_step < 1 || tile_offset < 0) throw Error{1, "bad prefilter tile range"};
    const int64_t ntiles = ceil_div(c.n, kThreads);
    if (tile_offset >= ntiles) return;
    const int64_t mine = (ntiles - 1 - tile_offset) / tile_step + 1;
    switch (c.dp / 2) {
        case 2: launch<2>(c, tile_offset, tile_step, mine, d_ext_sorted, st); break;
        case 4: launch<4>(c, tile_offset, tile_step, mine, d_ext_sorted, st); break;
        case 6: launch<6>(c, tile_offset, tile_step, mine, d_ext_sorted, st); break;
        case 8: launch<8>(c, tile_offset, tile_step, mine, d_ext_sorted, st); break;
        default: throw Error{1, "unsupported dimensionality"};
    }
}

}  // namespace sky
