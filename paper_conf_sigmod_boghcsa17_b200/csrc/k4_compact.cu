// k4_compact.cu — K4: from the per-point membership rows (complement of B_{p notin S}, Alg. 3 line 13)
// to (a) the row-major membership bitmap by point id and (b) the lattice of Fig. 1a (L151): for every
// subspace delta the ascending id list of S_delta(P).
//
// Input: rows of the S+ points in the tiled layout of K3: group g of 32 consecutive S+ points (id
// order), word w, lane l at rows32[g*W*32 + w*32 + l].  A warp loads one word of 32 points (128 B,
// coalesced) and transposes the 32x32 bit block with five shuffle stages, so that lane b holds the
// 32-point membership mask of subspace delta = 32w + b.  Counting pass -> 64-bit exclusive scan over
// (delta, chunk) -> scatter pass writing ids in ascending order.  HBM-bound.
#include <algorithm>

#include "ctx.cuh"

namespace sky {
namespace {

__device__ __forceinline__ uint32_t transpose32(uint32_t x, int lane) {
    const uint32_t masks[5] = {0x0000ffffu, 0x00ff00ffu, 0x0f0f0f0fu, 0x33333333u, 0x55555555u};
#pragma unroll
    for (int s = 0; s < 5; s++) {
        const int j = 16 >> s;
        const uint32_t lo = masks[s];
        const uint32_t y = __shfl_xor_sync(0xffffffffu, x, j);
        x = (lane & j) ? ((x & ~lo) | ((y >> j) & lo)) : ((x & lo) | ((y << j) & ~lo));
    }
    return x;  // bit l of lane b = bit b of the input of lane l
}

// Row-major membership by id: one block per (group of 32 points, chunk of up to 32 words).
__global__ void membership_kernel(const uint32_t *__restrict__ rows32, const int32_t *__restrict__ ext_ids, int64_t m,
                                  uint32_t W, uint32_t *__restrict__ membership) {
    __shared__ uint32_t tile[32][33];
    const int64_t g = blockIdx.x;
    const uint32_t wc = blockIdx.y * 32u;
    const uint32_t nw = min(32u, W - wc);
    const int tx = threadIdx.x & 31, ty = threadIdx.x >> 5;  // 32 x 8 threads
    for (uint32_t w = ty; w < nw; w += 8) tile[w][tx] = rows32[g * W * 32 + (int64_t)(wc + w) * 32 + tx];
    __syncthreads();
    for (int l = ty; l < 32; l += 8) {
        const int64_t j = g * 32 + l;
        if (j >= m) break;
        if ((uint32_t)tx < nw) membership[(int64_t)ext_ids[j] * W + wc + tx] = tile[tx][l];
    }
}

// Zero the rows of the points outside S+ (L101: they are in no skyline); one thread per word.
__global__ void zero_outside_kernel(const uint32_t *__restrict__ ext_id_flag, int64_t n, uint32_t W,
                                    uint32_t *__restrict__ membership) {
    const int64_t total = n * (int64_t)W;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x)
        if (!ext_id_flag[i / W]) membership[i] = 0u;
}

// counts[delta * nchunks + c] = |S_delta restricted to chunk c|.
template <int NWK>
__global__ void __launch_bounds__(NWK * 32) lattice_count_kernel(const uint32_t *__restrict__ rows32, int64_t m,
                                                               uint32_t W, int64_t nchunks,
                                                               uint64_t *__restrict__ counts) {
    __shared__ uint32_t red[NWK][32];
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int64_t c = blockIdx.x;
    const int64_t g = c * NWK + warp;
    for (uint32_t w = blockIdx.y; w < W; w += gridDim.y) {
        const uint32_t x = g * 32 + lane < m ? rows32[g * W * 32 + (int64_t)w * 32 + lane] : 0u;  // tail lanes unused
        red[warp][lane] = __popc(transpose32(x, lane));
        __syncthreads();
        if (warp == 0) {
            uint32_t s = 0;
#pragma unroll
            for (int k = 0; k < NWK; k++) s += red[k][lane];
            counts[((int64_t)w * 32 + lane) * nchunks + c] = s;
        }
        __syncthreads();
    }
}

// Scatter: warp = group of 32 tasks, lane = task.  After the transpose lane b holds the task mask of
// subspace delta = 32w + b and its segment offset; the warp then writes each non-empty subspace's ids with
// one coalesced store (the set lanes write consecutive addresses), instead of 32 lanes each appending to a
// different list (4-byte scattered stores: 8x sector write amplification, 58 ms at d = 16).
template <int NWK>
__global__ void __launch_bounds__(NWK * 32) lattice_scatter_kernel(const uint32_t *__restrict__ rows32, int64_t m,
                                                                 uint32_t W, int64_t nchunks,
                                                                 const uint64_t *__restrict__ base,
                                                                 const int32_t *__restrict__ ext_ids,
                                                                 int32_t *__restrict__ ids) {
    __shared__ uint32_t red[NWK][32];
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int64_t c = blockIdx.x;
    const int64_t g = c * NWK + warp;
    const int64_t j = g * 32 + lane;
    const int32_t my_id = j < m ? ext_ids[j] : 0;
    const uint32_t lt = (1u << lane) - 1u;
    for (uint32_t w = blockIdx.y; w < W; w += gridDim.y) {
        const uint32_t x = j < m ? rows32[g * W * 32 + (int64_t)w * 32 + lane] : 0u;  // tail lanes unused
        const uint32_t mask = transpose32(x, lane);  // lane b: tasks of the group in subspace 32w + b
        red[warp][lane] = __popc(mask);
        __syncthreads();
        uint64_t off = base[((int64_t)w * 32 + lane) * nchunks + c];
        for (int k = 0; k < warp; k++) off += red[k][lane];
        uint32_t nz = __ballot_sync(0xffffffffu, mask != 0u);
        while (nz) {
            const int b = __ffs(nz) - 1;
            nz &= nz - 1;
            const uint32_t mb = __shfl_sync(0xffffffffu, mask, b);
            const uint64_t ob = __shfl_sync(0xffffffffu, off, b);
            if ((mb >> lane) & 1u) ids[ob + __popc(mb & lt)] = my_id;
        }
        __syncthreads();
    }
}

__global__ void lattice_offsets_kernel(const uint64_t *__restrict__ base, const uint64_t *__restrict__ counts,
                                       int64_t nchunks, int64_t nsub, int64_t nentries, int64_t *__restrict__ offsets) {
    const int64_t delta = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (delta > nsub) return;
    if (delta < nsub) offsets[delta] = (int64_t)base[delta * nchunks];
    else offsets[delta] = (int64_t)(base[nentries - 1] + counts[nentries - 1]);
}

}  // namespace

void compact_membership(Ctx &c, const uint32_t *rows32, uint32_t *membership, cudaStream_t st) {
    SKY_CUDA(cudaMemsetAsync(membership, 0, sizeof(uint32_t) * (size_t)c.n * c.W, st));
    if (c.m == 0) return;
    dim3 grid((unsigned)ceil_div(c.m, 32), (unsigned)ceil_div(c.W, 32));
    membership_kernel<<<grid, 256, 0, st>>>(rows32, c.ext_ids.as<int32_t>(), c.m, c.W, membership);
    c.L.count++;
    SKY_LAUNCH_CHECK();
}

void membership_zero_outside(Ctx &c, uint32_t *membership, cudaStream_t st) {
    if (c.n == 0) return;
    const int64_t total = c.n * (int64_t)c.W;
    const unsigned blocks = (unsigned)std::min<int64_t>(ceil_div(total, 256), (int64_t)c.num_sms * 8);
    zero_outside_kernel<<<blocks, 256, 0, st>>>(c.ext_id_flag.as<uint32_t>(), c.n, c.W, membership);
    c.L.count++;
    SKY_LAUNCH_CHECK();
}

// Two calls: ids == nullptr computes counts/scan/offsets and *total_ids; then ids != nullptr scatters.
void compact_lattice(Ctx &c, const uint32_t *rows32, int64_t *offsets, int32_t *ids, int64_t *total_ids,
                     cudaStream_t st) {
    const int64_t nsub = (int64_t)1 << c.d;
    const int64_t ngroups = ceil_div(c.m, 32);
    const bool big = c.d > 12;
    const int nwk = big ? 32 : 8;
    const int64_t nchunks = ceil_div(ngroups > 0 ? ngroups : 1, nwk);
    const int64_t nentries = (int64_t)c.W * 32 * nchunks;  // >= nsub * nchunks
    const unsigned gy = (unsigned)std::min<int64_t>(c.W, big ? 64 : 16);
    dim3 grid((unsigned)nchunks, gy);
    if (ids == nullptr) {
        c.lat_counts.ensure(sizeof(uint64_t) * 2 * (size_t)nentries);
        c.scan64_tmp.ensure(scan_tmp_bytes(nentries));
        uint64_t *counts = c.lat_counts.as<uint64_t>();
        uint64_t *base = counts + nentries;
        if (c.m == 0) {
            SKY_CUDA(cudaMemsetAsync(counts, 0, sizeof(uint64_t) * 2 * (size_t)nentries, st));
        } else if (big) {
            lattice_count_kernel<32><<<grid, 32 * 32, 0, st>>>(rows32, c.m, c.W, nchunks, counts);
        } else {
            lattice_count_kernel<8><<<grid, 8 * 32, 0, st>>>(rows32, c.m, c.W, nchunks, counts);
        }
        if (c.m) {
            c.L.count++;
            SKY_LAUNCH_CHECK();
        }
        exclusive_scan_u64(counts, base, nentries, c.scan64_tmp.p, st, c.L);
        lattice_offsets_kernel<<<(unsigned)ceil_div(nsub + 1, 256), 256, 0, st>>>(base, counts, nchunks, nsub, nentries,
                                                                                 offsets);
        c.L.count++;
        SKY_LAUNCH_CHECK();
        int64_t tot = 0;
        SKY_CUDA(cudaMemcpyAsync(&tot, offsets + nsub, sizeof(int64_t), cudaMemcpyDeviceToHost, st));
        SKY_CUDA(cudaStreamSynchronize(st));
        *total_ids = tot;
        return;
    }
    if (c.m == 0) return;
    const uint64_t *base = c.lat_counts.as<uint64_t>() + nentries;
    if (big)
        lattice_scatter_kernel<32><<<grid, 32 * 32, 0, st>>>(rows32, c.m, c.W, nchunks, base, c.ext_ids.as<int32_t>(), ids);
    else
        lattice_scatter_kernel<8><<<grid, 8 * 32, 0, st>>>(rows32, c.m, c.W, nchunks, base, c.ext_ids.as<int32_t>(), ids);
    c.L.count++;
    SKY_LAUNCH_CHECK();
}

}  // namespace sky
