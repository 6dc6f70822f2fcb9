// k5_hashcube.cu — K5: the HashCube output of MDMC (Alg. 3 lines 1 and 13, L320; Appendix B.1,
// L1274-1282; Fig. 1b).  Each point p is represented by B_{p notin S} (2^d - 1 bits, bit delta-1 <=> p is
// dominated in delta, the shifted order of L84); the bitmask is cut into words of w bits and word k is
// hashed by h_k: key = the word, value = the ids of the points with that word.  A point whose word is
// all set (dominated in all w subspaces) is not stored (L1278).  Points outside S+(P) are dominated
// everywhere (L106) and never stored, so only the S+ rows of K3 are read.
//
// The hash maps are materialised as sorted arrays (reading H1): for every word k its distinct
// keys ascending, each with its ascending id list.  GPU construction, all HBM-bound:
//   items    one (word k, S+ point j) item per thread, k-major: composite key (k << w) | key (all-set words
//            get the sentinel nwords << w), value = id; the rows are read in K3's tiled layout (a warp
//            reads one word of 32 consecutive tasks: 128 B coalesced);
//   sort     stable LSD radix sort of the composites (w + log2(nwords+1) bits) -- stability keeps the
//            ids ascending within a key because items are generated in ascending id order;
//   unique   head flags -> exclusive scan -> per distinct composite: key, first item (key_offsets);
//   words    word_offsets[k] = lower_bound(distinct composites, k << w).
#include <algorithm>

#include "ctx.cuh"

namespace sky {
namespace {

__global__ void hc_items_kernel(const uint32_t *__restrict__ rows32, const int32_t *__restrict__ ext_ids, int64_t m,
                                uint32_t W, uint32_t nbits, uint32_t w, int64_t nwords, uint64_t *__restrict__ keys,
                                uint32_t *__restrict__ vals, unsigned long long *__restrict__ nvalid) {
    const int64_t total = nwords * m;
    const uint64_t sentinel = (uint64_t)nwords << w;
    unsigned long long cnt = 0;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x) {
        const int64_t k = i / m, j = i - k * m;
        const uint32_t b0 = (uint32_t)k * w + 1u;  // unshifted bit of the word's first subspace
        const uint32_t lo = b0 >> 5, sh = b0 & 31u;
        const uint32_t *row = rows32 + (j >> 5) * (int64_t)W * 32 + (j & 31);
        const uint64_t x0 = ~row[(int64_t)lo * 32];
        const uint64_t x1 = lo + 1 < W ? (uint64_t)(~row[(int64_t)(lo + 1) * 32]) : 0ull;
        const uint64_t v = ((x1 << 32) | (x0 & 0xffffffffull)) >> sh;
        const uint32_t valid = min(w, nbits - (uint32_t)k * w);
        const uint64_t full = (1ull << valid) - 1ull;
        const uint64_t key = v & full;
        const bool keep = key != full;
        keys[i] = keep ? (((uint64_t)k << w) | key) : sentinel;
        vals[i] = (uint32_t)ext_ids[j];
        cnt += keep;
    }
    for (int o = 16; o; o >>= 1) cnt += __shfl_xor_sync(0xffffffffu, cnt, o);
    if ((threadIdx.x & 31) == 0 && cnt) atomicAdd(nvalid, cnt);
}

__global__ void hc_heads_kernel(const uint64_t *__restrict__ keys, int64_t nvalid, uint32_t *__restrict__ head) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < nvalid; i += (int64_t)gridDim.x * blockDim.x)
        head[i] = (i == 0 || keys[i] != keys[i - 1]) ? 1u : 0u;
}

__global__ void hc_unique_kernel(const uint64_t *__restrict__ keys, const uint32_t *__restrict__ head,
                                 const uint32_t *__restrict__ idx, int64_t nvalid, uint32_t w,
                                 uint64_t *__restrict__ ukeys, uint32_t *__restrict__ keys32,
                                 int64_t *__restrict__ key_offsets) {
    const uint64_t mask = (w >= 32) ? 0xffffffffull : ((1ull << w) - 1ull);
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < nvalid; i += (int64_t)gridDim.x * blockDim.x) {
        if (!head[i]) continue;
        const uint32_t u = idx[i];
        ukeys[u] = keys[i];
        keys32[u] = (uint32_t)(keys[i] & mask);
        key_offsets[u] = i;
    }
}

__global__ void hc_words_kernel(const uint64_t *__restrict__ ukeys, int64_t nkeys, int64_t nwords, uint32_t w,
                                int64_t nvalid, int64_t *__restrict__ word_offsets, int64_t *__restrict__ key_offsets) {
    const int64_t k = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (k > nwords) return;
    const uint64_t target = (uint64_t)k << w;
    int64_t lo = 0, hi = nkeys;
    while (lo < hi) {
        const int64_t mid = (lo + hi) >> 1;
        if (ukeys[mid] < target) lo = mid + 1;
        else hi = mid;
    }
    word_offsets[k] = lo;
    if (k == nwords) key_offsets[nkeys] = nvalid;
}

unsigned grid_for(int64_t n, int threads, int sms) {
    const int64_t b = ceil_div(n > 0 ? n : 1, threads);
    return (unsigned)std::min<int64_t>(b, (int64_t)sms * 16);
}

int bitlen(uint64_t x) {
    int b = 0;
    while (x) {
        b++;
        x >>= 1;
    }
    return b;
}

}  // namespace

int64_t hashcube_words(int d, uint32_t w) { return ceil_div(((int64_t)1 << d) - 1, (int64_t)w); }

void hashcube_build(Ctx &c, const uint32_t *rows32, uint32_t w, cudaStream_t st) {
    if (!c.ext_ready) throw Error{1, "HashCube before the extended skyline is installed"};
    if (w < 1 || w > 32) throw Error{1, "HashCube word length w must be in [1, 32]"};
    const int64_t nwords = hashcube_words(c.d, w);
    const int64_t m = c.m;
    const int64_t N = nwords * m;
    if (N >= ((int64_t)1 << 32)) throw Error{3, "HashCube: (words x S+ points) exceeds 2^32 items"};
    HashCubeState &h = c.hc;
    h.w = w;
    h.nwords = nwords;
    h.nvalid = 0;
    h.nkeys = 0;
    h.woff.ensure(sizeof(int64_t) * (size_t)(nwords + 1));
    h.koff.ensure(sizeof(int64_t) * 8);
    if (N == 0) {
        SKY_CUDA(cudaMemsetAsync(h.woff.p, 0, sizeof(int64_t) * (size_t)(nwords + 1), st));
        SKY_CUDA(cudaMemsetAsync(h.koff.p, 0, sizeof(int64_t), st));
        h.built = true;
        return;
    }
    h.keys.ensure(sizeof(uint64_t) * (size_t)N);
    h.vals.ensure(sizeof(uint32_t) * (size_t)N);
    h.keys_alt.ensure(sizeof(uint64_t) * (size_t)N);
    h.vals_alt.ensure(sizeof(uint32_t) * (size_t)N);
    h.counts.ensure(sizeof(uint32_t) * radix_scratch_counts(N));
    const int64_t scan_n = std::max<int64_t>((int64_t)radix_scratch_counts(N), N);
    h.scan_tmp.ensure(scan_tmp_bytes(scan_n));
    h.nvalid_dev.ensure(sizeof(unsigned long long));
    SKY_CUDA(cudaMemsetAsync(h.nvalid_dev.p, 0, sizeof(unsigned long long), st));
    const uint32_t nbits = (uint32_t)(((int64_t)1 << c.d) - 1);
    hc_items_kernel<<<grid_for(N, 256, c.num_sms), 256, 0, st>>>(rows32, c.ext_ids.as<int32_t>(), m, c.W, nbits, w,
                                                                nwords, h.keys.as<uint64_t>(), h.vals.as<uint32_t>(),
                                                                h.nvalid_dev.as<unsigned long long>());
    c.L.count++;
    SKY_LAUNCH_CHECK();
    const int bits = (int)w + bitlen((uint64_t)nwords);
    radix_sort_u64(h.keys.as<uint64_t>(), h.vals.as<uint32_t>(), N, bits, h.keys_alt.as<uint64_t>(),
                   h.vals_alt.as<uint32_t>(), h.counts.as<uint32_t>(), h.scan_tmp.p, st, c.L);
    unsigned long long nvalid = 0;
    SKY_CUDA(cudaMemcpyAsync(&nvalid, h.nvalid_dev.p, sizeof(nvalid), cudaMemcpyDeviceToHost, st));
    SKY_CUDA(cudaStreamSynchronize(st));
    h.nvalid = (int64_t)nvalid;
    // head flags and their scan live in the (now free) ping-pong key buffer
    uint32_t *head = reinterpret_cast<uint32_t *>(h.keys_alt.p);
    uint32_t *idx = head + N;
    int64_t nkeys = 0;
    if (nvalid > 0) {
        hc_heads_kernel<<<grid_for(nvalid, 256, c.num_sms), 256, 0, st>>>(h.keys.as<uint64_t>(), nvalid, head);
        c.L.count++;
        SKY_LAUNCH_CHECK();
        exclusive_scan_u32(head, idx, nvalid, h.scan_tmp.p, st, c.L);
        uint32_t last[2] = {0, 0};
        SKY_CUDA(cudaMemcpyAsync(&last[0], idx + nvalid - 1, sizeof(uint32_t), cudaMemcpyDeviceToHost, st));
        SKY_CUDA(cudaMemcpyAsync(&last[1], head + nvalid - 1, sizeof(uint32_t), cudaMemcpyDeviceToHost, st));
        SKY_CUDA(cudaStreamSynchronize(st));
        nkeys = (int64_t)last[0] + last[1];
    }
    h.nkeys = nkeys;
    h.ukeys.ensure(sizeof(uint64_t) * (size_t)std::max<int64_t>(nkeys, 1));
    h.keys32.ensure(sizeof(uint32_t) * (size_t)std::max<int64_t>(nkeys, 1));
    h.koff.ensure(sizeof(int64_t) * (size_t)(nkeys + 1));
    if (nvalid > 0) {
        hc_unique_kernel<<<grid_for(nvalid, 256, c.num_sms), 256, 0, st>>>(h.keys.as<uint64_t>(), head, idx, nvalid, w,
                                                                          h.ukeys.as<uint64_t>(), h.keys32.as<uint32_t>(),
                                                                          h.koff.as<int64_t>());
        c.L.count++;
        SKY_LAUNCH_CHECK();
    }
    hc_words_kernel<<<(unsigned)ceil_div(nwords + 1, 256), 256, 0, st>>>(h.ukeys.as<uint64_t>(), nkeys, nwords, w,
                                                                       (int64_t)nvalid, h.woff.as<int64_t>(),
                                                                       h.koff.as<int64_t>());
    c.L.count++;
    SKY_LAUNCH_CHECK();
    h.built = true;
}

}  // namespace sky
