// sort_scan.cu — hand-written scan and stable LSD radix sort used by the preparation phase
// (key-sum order of Λ2 for the prefilter; per-dimension dense ranks for the K2 codes).
#include "common.cuh"

namespace sky {

namespace {

constexpr int kScanThreads = 512;
constexpr int kScanIpt = 8;
constexpr int kScanTile = kScanThreads * kScanIpt;  // 4096 items per block

template <typename T>
__device__ __forceinline__ T block_exclusive_sum(T v, T *total) {
    __shared__ T warp_sums[kScanThreads / 32];
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    T x = v;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        T y = __shfl_up_sync(0xffffffffu, x, o);
        if (lane >= o) x += y;
    }
    if (lane == 31) warp_sums[warp] = x;
    __syncthreads();
    if (warp == 0) {
        T s = lane < kScanThreads / 32 ? warp_sums[lane] : T(0);
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            T y = __shfl_up_sync(0xffffffffu, s, o);
            if (lane >= o) s += y;
        }
        if (lane < kScanThreads / 32) warp_sums[lane] = s;
    }
    __syncthreads();
    T warp_prefix = warp > 0 ? warp_sums[warp - 1] : T(0);
    if (total) *total = warp_sums[kScanThreads / 32 - 1];
    __syncthreads();
    return warp_prefix + x - v;
}

template <typename T>
__global__ void scan_reduce_kernel(const T *__restrict__ in, T *__restrict__ partial, int64_t n) {
    const int64_t base = (int64_t)blockIdx.x * kScanTile + (int64_t)threadIdx.x * kScanIpt;
    T s = 0;
#pragma unroll
    for (int k = 0; k < kScanIpt; k++)
        if (base + k < n) s += in[base + k];
    T total;
    block_exclusive_sum<T>(s, &total);
    if (threadIdx.x == 0) partial[blockIdx.x] = total;
}

template <typename T>
__global__ void scan_down_kernel(const T *in, T *out, const T *__restrict__ partial, int64_t n) {
    const int64_t base = (int64_t)blockIdx.x * kScanTile + (int64_t)threadIdx.x * kScanIpt;
    T v[kScanIpt];
    T s = 0;
#pragma unroll
    for (int k = 0; k < kScanIpt; k++) {
        v[k] = base + k < n ? in[base + k] : T(0);
        s += v[k];
    }
    T pre = block_exclusive_sum<T>(s, nullptr) + (partial ? partial[blockIdx.x] : T(0));
#pragma unroll
    for (int k = 0; k < kScanIpt; k++) {
        if (base + k < n) out[base + k] = pre;
        pre += v[k];
    }
}

template <typename T>
void exclusive_scan_impl(const T *in, T *out, int64_t n, T *tmp, cudaStream_t st, Launches &L) {
    if (n <= 0) return;
    const int64_t nb = ceil_div(n, kScanTile);
    if (nb == 1) {
        scan_down_kernel<T><<<1, kScanThreads, 0, st>>>(in, out, nullptr, n);
        L.count++;
        SKY_LAUNCH_CHECK();
        return;
    }
    T *partial = tmp;
    T *next_tmp = tmp + nb;
    scan_reduce_kernel<T><<<(unsigned)nb, kScanThreads, 0, st>>>(in, partial, n);
    L.count++;
    SKY_LAUNCH_CHECK();
    exclusive_scan_impl<T>(partial, partial, nb, next_tmp, st, L);
    scan_down_kernel<T><<<(unsigned)nb, kScanThreads, 0, st>>>(in, out, partial, n);
    L.count++;
    SKY_LAUNCH_CHECK();
}

// ------------------------------------------------------------------------------------ radix sort
constexpr int kRsThreads = 256;
constexpr int kRsIpt = 8;
constexpr int kRsTile = kRsThreads * kRsIpt;
constexpr int kRsWarps = kRsThreads / 32;

__global__ void radix_hist_kernel(const uint64_t *__restrict__ keys, int64_t n, int shift,
                                  uint32_t *__restrict__ counts, int nblocks) {
    __shared__ uint32_t hist[256];
    for (int i = threadIdx.x; i < 256; i += blockDim.x) hist[i] = 0;
    __syncthreads();
    const int64_t base = (int64_t)blockIdx.x * kRsTile;
    for (int k = threadIdx.x; k < kRsTile; k += kRsThreads) {
        int64_t idx = base + k;
        if (idx < n) atomicAdd(&hist[(uint32_t)(keys[idx] >> shift) & 0xffu], 1u);
    }
    __syncthreads();
    for (int i = threadIdx.x; i < 256; i += blockDim.x) counts[(int64_t)i * nblocks + blockIdx.x] = hist[i];
}

__global__ void radix_scatter_kernel(const uint64_t *__restrict__ keys, const uint32_t *__restrict__ vals,
                                     uint64_t *__restrict__ keys_out, uint32_t *__restrict__ vals_out,
                                     int64_t n, int shift, const uint32_t *__restrict__ offsets, int nblocks) {
    __shared__ uint32_t run[257];
    __shared__ uint32_t wcnt[kRsWarps][257];
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    for (int i = threadIdx.x; i < 256; i += blockDim.x) run[i] = offsets[(int64_t)i * nblocks + blockIdx.x];
    for (int i = threadIdx.x; i < kRsWarps * 257; i += blockDim.x) (&wcnt[0][0])[i] = 0;
    __syncthreads();
    const uint32_t lt_mask = (1u << lane) - 1u;
    const int64_t base = (int64_t)blockIdx.x * kRsTile;
    for (int r = 0; r < kRsIpt; r++) {
        const int64_t idx = base + (int64_t)r * kRsThreads + threadIdx.x;
        const bool valid = idx < n;
        uint64_t key = 0;
        uint32_t val = 0;
        uint32_t dg = 256;
        if (valid) {
            key = keys[idx];
            val = vals[idx];
            dg = (uint32_t)(key >> shift) & 0xffu;
        }
        const uint32_t peers = __match_any_sync(0xffffffffu, dg);
        const uint32_t wrank = __popc(peers & lt_mask);
        const uint32_t tag = (uint32_t)(r + 1) << 16;
        if (wrank == 0) wcnt[warp][dg] = tag | (uint32_t)__popc(peers);
        __syncthreads();
        uint32_t pre = 0;
        for (int w = 0; w < warp; w++) {
            uint32_t e = wcnt[w][dg];
            if ((e & 0xffff0000u) == tag) pre += e & 0xffffu;
        }
        const uint32_t pos = run[dg] + pre + wrank;
        __syncthreads();
        if (wrank == 0) atomicAdd(&run[dg], (uint32_t)__popc(peers));
        if (valid) {
            keys_out[pos] = key;
            vals_out[pos] = val;
        }
        __syncthreads();
    }
}

}  // namespace

size_t scan_tmp_bytes(int64_t n) {
    size_t total = 0;
    int64_t m = n;
    while (m > 1) {
        m = ceil_div(m, kScanTile);
        total += (size_t)m * sizeof(uint64_t);
    }
    return total + 64;
}

void exclusive_scan_u32(const uint32_t *in, uint32_t *out, int64_t n, void *tmp, cudaStream_t st, Launches &L) {
    exclusive_scan_impl<uint32_t>(in, out, n, (uint32_t *)tmp, st, L);
}

void exclusive_scan_u64(const uint64_t *in, uint64_t *out, int64_t n, void *tmp, cudaStream_t st, Launches &L) {
    exclusive_scan_impl<uint64_t>(in, out, n, (uint64_t *)tmp, st, L);
}

size_t radix_scratch_counts(int64_t n) { return (size_t)256 * (size_t)ceil_div(n > 0 ? n : 1, kRsTile); }

void radix_sort_u64(uint64_t *keys, uint32_t *vals, int64_t n, int bits, uint64_t *keys_alt,
                    uint32_t *vals_alt, uint32_t *counts, void *scan_tmp, cudaStream_t st, Launches &L) {
    if (n <= 1) return;
    const int nblocks = (int)ceil_div(n, kRsTile);
    const int passes = (bits + 7) / 8;
    uint64_t *kin = keys, *kout = keys_alt;
    uint32_t *vin = vals, *vout = vals_alt;
    for (int p = 0; p < passes; p++) {
        const int shift = 8 * p;
        radix_hist_kernel<<<nblocks, kRsThreads, 0, st>>>(kin, n, shift, counts, nblocks);
        L.count++;
        SKY_LAUNCH_CHECK();
        exclusive_scan_u32(counts, counts, (int64_t)256 * nblocks, scan_tmp, st, L);
        radix_scatter_kernel<<<nblocks, kRsThreads, 0, st>>>(kin, vin, kout, vout, n, shift, counts, nblocks);
        L.count++;
        SKY_LAUNCH_CHECK();
        uint64_t *tk = kin; kin = kout; kout = tk;
        uint32_t *tv = vin; vin = vout; vout = tv;
    }
    if (kin != keys) {
        SKY_CUDA(cudaMemcpyAsync(keys, kin, sizeof(uint64_t) * n, cudaMemcpyDeviceToDevice, st));
        SKY_CUDA(cudaMemcpyAsync(vals, vin, sizeof(uint32_t) * n, cudaMemcpyDeviceToDevice, st));
    }
}

}  // namespace sky
