// k4_compact.cu — K4: from the per-point membership rows (complement of B_{p notin S}, Alg. 3 line 13)
// to (a) the row-major membership bitmap by point id and (b) the lattice of Fig. 1a (L156): for every
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

// Zero the rows of the points outside S+ (L106: they are in no skyline); one thread per word.
__global__ void zero_outside_kernel(const uint32_t *__restrict__ ext_id_flag, int64_t n, uint32_t W,
                                    uint32_t *__restrict__ membership) {
    const int64_t total = n * (int64_t)W;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x)
        if (!ext_id_flag[i / W]) membership[i] = 0u;
}

// Lattice (CSR per subspace, ascending ids).  A block = NWK groups of 32 tasks ("chunk" c); per word w of
// the rows, lane b of a warp holds (after the transpose) the task mask of subspace delta = 32w + b.
// Counts are stored chunk-major, counts[c * NS + delta] (NS = 32 W >= 2^d), so a warp's 32 subspaces are 32
// consecutive entries (coalesced); the offset of (delta, c) is doff[delta] + colpre[c * NS + delta], where
// colpre is the prefix over chunks per subspace and doff the exclusive scan of the per-subspace totals.
// UNR words per iteration keep several 128-byte row loads in flight per warp.
constexpr int kUnr = 4;

template <int NWK>
__global__ void __launch_bounds__(NWK * 32) lattice_count_kernel(const uint32_t *__restrict__ rows32, int64_t m,
                                                               uint32_t W, uint64_t *__restrict__ counts) {
    __shared__ uint32_t red[kUnr][NWK][32];
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int64_t c = blockIdx.x;
    const int64_t g = c * NWK + warp;
    const int64_t NS = (int64_t)W * 32;
    const bool live = g * 32 + lane < m;  // tail lanes unused
    for (uint32_t w0 = blockIdx.y * kUnr; w0 < W; w0 += gridDim.y * kUnr) {
        uint32_t x[kUnr];
#pragma unroll
        for (int u = 0; u < kUnr; u++)
            x[u] = live && w0 + u < W ? rows32[g * W * 32 + (int64_t)(w0 + u) * 32 + lane] : 0u;
#pragma unroll
        for (int u = 0; u < kUnr; u++) red[u][warp][lane] = __popc(transpose32(x[u], lane));
        __syncthreads();
        if (warp < kUnr && w0 + warp < W) {
            uint32_t s = 0;
#pragma unroll
            for (int k = 0; k < NWK; k++) s += red[warp][k][lane];
            counts[c * NS + (int64_t)(w0 + warp) * 32 + lane] = s;
        }
        __syncthreads();
    }
}

// colpre[c * NS + delta] = sum of counts of chunks < c; tot[delta] = sum over all chunks.  Thread = subspace.
__global__ void lattice_colscan_kernel(const uint64_t *__restrict__ counts, int64_t nchunks, int64_t NS,
                                       uint64_t *__restrict__ colpre, uint64_t *__restrict__ tot) {
    const int64_t delta = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (delta >= NS) return;
    uint64_t run = 0;
    int64_t c = 0;
    for (; c + 4 <= nchunks; c += 4) {
        uint64_t v[4];
#pragma unroll
        for (int u = 0; u < 4; u++) v[u] = counts[(c + u) * NS + delta];
#pragma unroll
        for (int u = 0; u < 4; u++) {
            colpre[(c + u) * NS + delta] = run;
            run += v[u];
        }
    }
    for (; c < nchunks; c++) {
        const uint64_t v = counts[c * NS + delta];
        colpre[c * NS + delta] = run;
        run += v;
    }
    tot[delta] = run;
}

// Scatter: warp = group of 32 tasks, lane = task.  After the transpose lane b holds the task mask of
// subspace delta = 32w + b and its segment offset; the warp then writes each non-empty subspace's ids with
// one coalesced store (the set lanes write consecutive addresses), instead of 32 lanes each appending to a
// different list (4-byte scattered stores: 8x sector write amplification).
template <int NWK>
__global__ void __launch_bounds__(NWK * 32) lattice_scatter_kernel(const uint32_t *__restrict__ rows32, int64_t m,
                                                                 uint32_t W, const uint64_t *__restrict__ colpre,
                                                                 const uint64_t *__restrict__ doff,
                                                                 const int32_t *__restrict__ ext_ids,
                                                                 int32_t *__restrict__ ids) {
    __shared__ uint32_t red[kUnr][NWK][32];
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int64_t c = blockIdx.x;
    const int64_t g = c * NWK + warp;
    const int64_t NS = (int64_t)W * 32;
    const int64_t j = g * 32 + lane;
    const bool live = j < m;
    const int32_t my_id = live ? ext_ids[j] : 0;
    const uint32_t lt = (1u << lane) - 1u;
    for (uint32_t w0 = blockIdx.y * kUnr; w0 < W; w0 += gridDim.y * kUnr) {
        uint32_t mask[kUnr];
        uint64_t off[kUnr];
#pragma unroll
        for (int u = 0; u < kUnr; u++) {
            const uint32_t x = live && w0 + u < W ? rows32[g * W * 32 + (int64_t)(w0 + u) * 32 + lane] : 0u;
            mask[u] = transpose32(x, lane);  // lane b: tasks of the group in subspace 32(w0+u) + b
            red[u][warp][lane] = __popc(mask[u]);
            const int64_t delta = (int64_t)(w0 + u) * 32 + lane;
            off[u] = w0 + u < W ? doff[delta] + colpre[c * NS + delta] : 0;
        }
        __syncthreads();
#pragma unroll
        for (int u = 0; u < kUnr; u++) {
            for (int k = 0; k < warp; k++) off[u] += red[u][k][lane];
            uint32_t nz = __ballot_sync(0xffffffffu, mask[u] != 0u);
            while (nz) {
                const int b = __ffs(nz) - 1;
                nz &= nz - 1;
                const uint32_t mb = __shfl_sync(0xffffffffu, mask[u], b);
                const uint64_t ob = __shfl_sync(0xffffffffu, off[u], b);
                if ((mb >> lane) & 1u) ids[ob + __popc(mb & lt)] = my_id;
            }
        }
        __syncthreads();
    }
}

// Scatter for large subspace counts (d > 12: every (subspace, group) segment holds only a few ids, so the
// per-group scatter above issues one store per ~4 ids).  A block = 32 groups (1024 tasks); per word w each
// warp transposes its group's word into shared memory, then warp b takes subspace delta = 32w + b with
// lane = group: a warp prefix sum of the 32 group counts places the whole 1024-task segment of delta, and
// lane-parallel stores write it (one store instruction per ~32 x 4 ids).
__global__ void __launch_bounds__(1024) lattice_scatter32_kernel(const uint32_t *__restrict__ rows32, int64_t m,
                                                               uint32_t W, const uint64_t *__restrict__ colpre,
                                                               const uint64_t *__restrict__ doff,
                                                               const int32_t *__restrict__ ext_ids,
                                                               int32_t *__restrict__ ids) {
    __shared__ uint32_t M[32][33];  // [group][subspace bit]
    __shared__ int32_t sid[1024];
    extern __shared__ int32_t stage[];  // [32 warps][1024]: the warp's subspace segment, compacted
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int64_t c = blockIdx.x;
    const int64_t g = c * 32 + warp;
    const int64_t NS = (int64_t)W * 32;
    const int64_t j = g * 32 + lane;
    int32_t *seg = stage + warp * 1024;
    sid[threadIdx.x] = j < m ? ext_ids[j] : 0;
    const uint32_t *rowp = rows32 + g * W * 32 + lane;
    uint32_t x_next = j < m && blockIdx.y < W ? rowp[(int64_t)blockIdx.y * 32] : 0u;
    for (uint32_t w = blockIdx.y; w < W; w += gridDim.y) {
        const uint32_t x = x_next;  // this word was loaded during the previous iteration (latency hidden)
        const uint32_t wn = w + gridDim.y;
        x_next = j < m && wn < W ? rowp[(int64_t)wn * 32] : 0u;
        M[warp][lane] = transpose32(x, lane);  // lane b: tasks of group `warp` in subspace 32w + b
        __syncthreads();
        const uint32_t mg = M[lane][warp];     // tasks of group `lane` in subspace 32w + warp
        const uint32_t cnt = __popc(mg);
        uint32_t incl = cnt;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const uint32_t y = __shfl_up_sync(0xffffffffu, incl, o);
            if (lane >= o) incl += y;
        }
        const uint32_t total = __shfl_sync(0xffffffffu, incl, 31);
        // compact this subspace's ids of the 1024 tasks into the warp's stage (ascending: group, then bit) ...
        uint32_t mm = mg, o = incl - cnt;
        while (mm) {
            const int b = __ffs(mm) - 1;
            mm &= mm - 1;
            seg[o++] = sid[lane * 32 + b];
        }
        __syncwarp();
        // ... and write the segment with full-line coalesced stores
        const int64_t delta = (int64_t)w * 32 + warp;
        int32_t *dst = ids + doff[delta] + colpre[c * NS + delta];
        for (uint32_t i = lane; i < total; i += 32) dst[i] = seg[i];
        __syncthreads();
    }
}

// Multi-GPU placement of one shard's segments: all[r * nsub + delta] = count of subspace
// delta in shard r.  tot[delta] = the global count, pre[delta] = the counts of the shards before `rank`.
__global__ void lattice_place_kernel(const int64_t *__restrict__ all, int k, int rank, int64_t nsub, int64_t NS,
                                     uint64_t *__restrict__ tot, uint64_t *__restrict__ pre) {
    const int64_t delta = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (delta >= NS) return;
    uint64_t t = 0, p = 0;
    if (delta < nsub)
        for (int r = 0; r < k; r++) {
            const uint64_t v = (uint64_t)all[(int64_t)r * nsub + delta];
            if (r < rank) p += v;
            t += v;
        }
    tot[delta] = t;
    pre[delta] = p;
}

// doff[delta] += pre[delta]: the shard's segment of subspace delta starts after the earlier shards' ids
__global__ void lattice_shift_kernel(uint64_t *__restrict__ doff, const uint64_t *__restrict__ pre, int64_t NS) {
    const int64_t delta = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (delta < NS) doff[delta] += pre[delta];
}

__global__ void totals_out_kernel(const uint64_t *__restrict__ tot, int64_t nsub, int64_t *__restrict__ out) {
    const int64_t delta = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (delta < nsub) out[delta] = (int64_t)tot[delta];
}

// Membership rows of the tasks of one shard, by point id; the rows of the points outside S+ with ids in
// [zlo, zhi) are zeroed (each shard zeroes its own slice of ids).  `membership` may be host-mapped.
__global__ void membership_shard_kernel(const uint32_t *__restrict__ rows32, const int32_t *__restrict__ ext_ids,
                                        int64_t mr, uint32_t W, uint32_t *__restrict__ membership) {
    __shared__ uint32_t tile[32][33];
    const int64_t g = blockIdx.x;
    const uint32_t wc = blockIdx.y * 32u;
    const uint32_t nw = min(32u, W - wc);
    const int tx = threadIdx.x & 31, ty = threadIdx.x >> 5;
    for (uint32_t w = ty; w < nw; w += 8) tile[w][tx] = rows32[g * W * 32 + (int64_t)(wc + w) * 32 + tx];
    __syncthreads();
    for (int l = ty; l < 32; l += 8) {
        const int64_t j = g * 32 + l;
        if (j >= mr) break;
        if ((uint32_t)tx < nw) membership[(int64_t)ext_ids[j] * W + wc + tx] = tile[tx][l];
    }
}

__global__ void zero_outside_range_kernel(const uint32_t *__restrict__ ext_id_flag, int64_t lo, int64_t hi, uint32_t W,
                                          uint32_t *__restrict__ membership) {
    const int64_t total = (hi - lo) * (int64_t)W;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x)
        if (!ext_id_flag[lo + i / W]) membership[lo * (int64_t)W + i] = 0u;
}

__global__ void lattice_offsets_kernel(const uint64_t *__restrict__ doff, const uint64_t *__restrict__ tot,
                                       int64_t nsub, int64_t *__restrict__ offsets) {
    const int64_t delta = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (delta > nsub) return;
    offsets[delta] = delta < nsub ? (int64_t)doff[delta] : (int64_t)(doff[nsub - 1] + tot[nsub - 1]);
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

// Geometry of the lattice passes over the shard of S+ tasks [j0, j1) (j0 a multiple of 32).
struct LatGeo {
    int64_t nsub, mr, nchunks, NS, nentries;
    bool big;
    int nwk;
    dim3 grid;
    LatGeo(const Ctx &c, int64_t j0, int64_t j1) {
        nsub = (int64_t)1 << c.d;
        mr = j1 - j0;
        big = c.d > 12;
        nwk = big ? 32 : 8;
        const int64_t ngroups = ceil_div(mr, 32);
        nchunks = ceil_div(ngroups > 0 ? ngroups : 1, nwk);
        NS = (int64_t)c.W * 32;  // >= nsub
        nentries = NS * nchunks;
        const unsigned gy = (unsigned)std::min<int64_t>(ceil_div(c.W, kUnr), big ? 16 : 4);
        grid = dim3((unsigned)nchunks, gy);
    }
};

// scratch: counts, colpre [nentries] then tot, doff, pre [NS]
static uint64_t *lat_scratch(Ctx &c, const LatGeo &g) {
    c.lat_counts.ensure(sizeof(uint64_t) * (2 * (size_t)g.nentries + 3 * (size_t)g.NS));
    return c.lat_counts.as<uint64_t>();
}

// Count pass of a shard: per (chunk, subspace) counts, the per-subspace prefix over the shard's chunks (kept in
// the context for the scatter) and the shard's per-subspace totals (written to d_totals[nsub] if non-null).
void lattice_count_shard(Ctx &c, const uint32_t *rows32, int64_t j0, int64_t j1, int64_t *d_totals, cudaStream_t st) {
    if (j0 < 0 || j1 > c.m || (j0 & 31) || j1 < j0) throw Error{1, "bad lattice shard range"};
    const LatGeo g(c, j0, j1);
    uint64_t *counts = lat_scratch(c, g), *colpre = counts + g.nentries, *tot = colpre + g.nentries;
    const uint32_t *rows = rows32 + (j0 / 32) * (int64_t)c.W * 32;
    if (g.mr == 0) {
        SKY_CUDA(cudaMemsetAsync(counts, 0, sizeof(uint64_t) * (size_t)g.nentries, st));
    } else {
        if (g.big)
            lattice_count_kernel<32><<<g.grid, 32 * 32, 0, st>>>(rows, g.mr, c.W, counts);
        else
            lattice_count_kernel<8><<<g.grid, 8 * 32, 0, st>>>(rows, g.mr, c.W, counts);
        c.L.count++;
        SKY_LAUNCH_CHECK();
    }
    lattice_colscan_kernel<<<(unsigned)ceil_div(g.NS, 128), 128, 0, st>>>(counts, g.nchunks, g.NS, colpre, tot);
    c.L.count++;
    SKY_LAUNCH_CHECK();
    if (d_totals) {
        totals_out_kernel<<<(unsigned)ceil_div(g.nsub, 256), 256, 0, st>>>(tot, g.nsub, d_totals);
        c.L.count++;
        SKY_LAUNCH_CHECK();
    }
}

// Scatter pass of a shard after lattice_count_shard: all_totals[k][nsub] are the totals of every shard (rank r
// covers the r-th task range in S+ order, so its ids of subspace delta follow those of ranks < r).  Writes the
// global offsets[nsub + 1] (nullable) and the shard's ids at their global positions of ids[] (device or
// host-mapped memory; ids of other shards are not touched).  Returns the global id count.
int64_t lattice_scatter_shard(Ctx &c, const uint32_t *rows32, int64_t j0, int64_t j1, const int64_t *all_totals, int k,
                              int rank, int64_t *offsets, int32_t *ids, cudaStream_t st) {
    const LatGeo g(c, j0, j1);
    uint64_t *counts = lat_scratch(c, g), *colpre = counts + g.nentries, *tot = colpre + g.nentries;
    uint64_t *doff = tot + g.NS, *pre = doff + g.NS;
    (void)counts;
    c.scan64_tmp.ensure(scan_tmp_bytes(g.NS));
    // global totals -> tot (the shard's own totals are no longer needed), the earlier shards' counts -> pre
    lattice_place_kernel<<<(unsigned)ceil_div(g.NS, 256), 256, 0, st>>>(all_totals, k, rank, g.nsub, g.NS, tot, pre);
    c.L.count++;
    SKY_LAUNCH_CHECK();
    exclusive_scan_u64(tot, doff, g.NS, c.scan64_tmp.p, st, c.L);
    if (offsets) {
        lattice_offsets_kernel<<<(unsigned)ceil_div(g.nsub + 1, 256), 256, 0, st>>>(doff, tot, g.nsub, offsets);
        c.L.count++;
        SKY_LAUNCH_CHECK();
    }
    int64_t total = 0;
    {
        uint64_t last[2];
        SKY_CUDA(cudaMemcpyAsync(&last[0], doff + g.nsub - 1, sizeof(uint64_t), cudaMemcpyDeviceToHost, st));
        SKY_CUDA(cudaMemcpyAsync(&last[1], tot + g.nsub - 1, sizeof(uint64_t), cudaMemcpyDeviceToHost, st));
        SKY_CUDA(cudaStreamSynchronize(st));
        total = (int64_t)(last[0] + last[1]);
    }
    if (g.mr == 0 || !ids) return total;
    if (k > 1 || rank > 0) {
        lattice_shift_kernel<<<(unsigned)ceil_div(g.NS, 256), 256, 0, st>>>(doff, pre, g.NS);
        c.L.count++;
        SKY_LAUNCH_CHECK();
    }
    const uint32_t *rows = rows32 + (j0 / 32) * (int64_t)c.W * 32;
    const int32_t *eid = c.ext_ids.as<int32_t>() + j0;
    if (g.big) {
        const int smem = 32 * 1024 * (int)sizeof(int32_t);
        SKY_CUDA(cudaFuncSetAttribute(lattice_scatter32_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
        lattice_scatter32_kernel<<<dim3((unsigned)g.nchunks, (unsigned)std::min<int64_t>(c.W, 64)), 1024, smem, st>>>(
            rows, g.mr, c.W, colpre, doff, eid, ids);
    } else {
        lattice_scatter_kernel<8><<<g.grid, 8 * 32, 0, st>>>(rows, g.mr, c.W, colpre, doff, eid, ids);
    }
    c.L.count++;
    SKY_LAUNCH_CHECK();
    return total;
}

// Single-GPU lattice: the whole of S+ as one shard.  Two calls: ids == nullptr computes counts/scan/offsets and
// *total_ids; then ids != nullptr scatters.
void compact_lattice(Ctx &c, const uint32_t *rows32, int64_t *offsets, int32_t *ids, int64_t *total_ids,
                     cudaStream_t st) {
    const LatGeo g(c, 0, c.m);
    if (ids == nullptr) {
        lattice_count_shard(c, rows32, 0, c.m, nullptr, st);
        uint64_t *counts = lat_scratch(c, g), *colpre = counts + g.nentries, *tot = colpre + g.nentries;
        uint64_t *doff = tot + g.NS;
        c.scan64_tmp.ensure(scan_tmp_bytes(g.NS));
        exclusive_scan_u64(tot, doff, g.NS, c.scan64_tmp.p, st, c.L);
        lattice_offsets_kernel<<<(unsigned)ceil_div(g.nsub + 1, 256), 256, 0, st>>>(doff, tot, g.nsub, offsets);
        c.L.count++;
        SKY_LAUNCH_CHECK();
        int64_t tot_ids = 0;
        SKY_CUDA(cudaMemcpyAsync(&tot_ids, offsets + g.nsub, sizeof(int64_t), cudaMemcpyDeviceToHost, st));
        SKY_CUDA(cudaStreamSynchronize(st));
        *total_ids = tot_ids;
        return;
    }
    if (c.m == 0) return;
    uint64_t *counts = lat_scratch(c, g), *colpre = counts + g.nentries, *tot = colpre + g.nentries;
    uint64_t *doff = tot + g.NS;
    (void)counts;
    if (g.big) {
        const int smem = 32 * 1024 * (int)sizeof(int32_t);
        SKY_CUDA(cudaFuncSetAttribute(lattice_scatter32_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
        lattice_scatter32_kernel<<<dim3((unsigned)g.nchunks, (unsigned)std::min<int64_t>(c.W, 64)), 1024, smem, st>>>(
            rows32, c.m, c.W, colpre, doff, c.ext_ids.as<int32_t>(), ids);
    } else {
        lattice_scatter_kernel<8><<<g.grid, 8 * 32, 0, st>>>(rows32, c.m, c.W, colpre, doff, c.ext_ids.as<int32_t>(), ids);
    }
    c.L.count++;
    SKY_LAUNCH_CHECK();
}

// Membership by id of the shard [j0, j1) of S+ tasks, and zero rows for the points outside S+ whose ids lie in
// [zlo, zhi).  `membership` [n][W] may be device or host-mapped memory; nothing else of it is touched.
void compact_membership_shard(Ctx &c, const uint32_t *rows32, int64_t j0, int64_t j1, int64_t zlo, int64_t zhi,
                              uint32_t *membership, cudaStream_t st) {
    if (j0 < 0 || j1 > c.m || (j0 & 31) || j1 < j0 || zlo < 0 || zhi > c.n || zhi < zlo)
        throw Error{1, "bad membership shard range"};
    if (zhi > zlo) {
        const int64_t total = (zhi - zlo) * (int64_t)c.W;
        const unsigned blocks = (unsigned)std::min<int64_t>(ceil_div(total, 256), (int64_t)c.num_sms * 8);
        zero_outside_range_kernel<<<blocks, 256, 0, st>>>(c.ext_id_flag.as<uint32_t>(), zlo, zhi, c.W, membership);
        c.L.count++;
        SKY_LAUNCH_CHECK();
    }
    if (j1 == j0) return;
    dim3 grid((unsigned)ceil_div(j1 - j0, 32), (unsigned)ceil_div(c.W, 32));
    membership_shard_kernel<<<grid, 256, 0, st>>>(rows32 + (j0 / 32) * (int64_t)c.W * 32, c.ext_ids.as<int32_t>() + j0,
                                                  j1 - j0, c.W, membership);
    c.L.count++;
    SKY_LAUNCH_CHECK();
}

}  // namespace sky
