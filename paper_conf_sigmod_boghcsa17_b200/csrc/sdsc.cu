// sdsc.cu — the SDSC template (single-device-single-cuboid, Alg. 2) on the GPU: the paper's
// lattice-based alternative to MDMC, built as an in-repo comparator.
//
// Top-down lattice traversal over extended skylines (Alg. 2):
//   line 2   L[full] <- S_full(P), L+[full] <- S+_full(P) \ S_full(P)        (input: S+(P) from K1)
//   line 3-4 for every level l = d-1 .. 1, all cuboids delta of the level in ONE batched pass (the GPU is
//            the "device"; the paper's cross-device task parallelism of line 4 becomes segment parallelism)
//   line 5   parent = the immediate superset delta' with the smallest |L[delta']| + |L+[delta']| (reading S1)
//   line 6   L[delta], L+[delta] from the parent's S+ list, by a parallel skyline over the cuboid's input.
// The parallel skyline (the "hook", L296-300) is a sorted prefix scan: the cuboid's points are sorted by the
// exact key sum_{i in delta} ord_i (only a point with a strictly smaller key can dominate, Λ2 restricted to
// delta), and each point is tested against the prefix before it, tile by tile through shared memory.
// Everything lives in the index space of S+(P) (j, ascending = ascending id): S+_delta(P) is a subset of
// S+(P) for every delta, so lists are ascending j sequences.
#include <algorithm>
#include <vector>

#include "ctx.cuh"

namespace sky {
namespace {

constexpr int kSkyThreads = 256;

// item e of the level belongs to segment k = upper_bound(seg_off, e) - 1
__device__ __forceinline__ int find_seg(const int64_t *__restrict__ seg_off, int nseg, int64_t e) {
    int lo = 0, hi = nseg;  // seg_off[lo] <= e < seg_off[hi]
    while (hi - lo > 1) {
        const int mid = (lo + hi) >> 1;
        if (seg_off[mid] <= e) lo = mid;
        else hi = mid;
    }
    return lo;
}

// Gather the cuboids' inputs (the parents' S+ lists) and form the sort keys (segment, key_delta).
__global__ void sdsc_gather_kernel(const uint32_t *__restrict__ prev, const int64_t *__restrict__ src_off,
                                   const int64_t *__restrict__ seg_off, const uint32_t *__restrict__ seg_delta,
                                   int nseg, int64_t total, const uint32_t *__restrict__ p_ord, int d,
                                   uint32_t *__restrict__ items, uint64_t *__restrict__ keys,
                                   uint32_t *__restrict__ vals) {
    for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < total; e += (int64_t)gridDim.x * blockDim.x) {
        const int k = find_seg(seg_off, nseg, e);
        const uint32_t j = prev ? (prev[src_off[k] + (e - seg_off[k])] & 0x7fffffffu) : (uint32_t)e;
        const uint32_t delta = seg_delta[k];
        uint64_t key = 0;
        for (int i = 0; i < d; i++)
            if ((delta >> i) & 1u) key += p_ord[(int64_t)j * d + i];
        items[e] = j;
        keys[e] = ((uint64_t)k << 36) | key;
        vals[e] = (uint32_t)e;
    }
}

// Skyline of every segment in delta: thread = item (sorted position r), scans the items of its segment
// sorted before it.  status: 0 = in S_delta, 1 = in S+_delta \ S_delta, 2 = not in S+_delta.
__global__ void __launch_bounds__(kSkyThreads) sdsc_sky_kernel(const uint32_t *__restrict__ items,
                                                                const uint32_t *__restrict__ perm,
                                                                const int64_t *__restrict__ seg_off,
                                                                const uint32_t *__restrict__ seg_delta, int nseg,
                                                                int64_t total, const uint32_t *__restrict__ p_ord,
                                                                int d, uint8_t *__restrict__ status) {
    __shared__ uint32_t tile[kSkyThreads][kMaxD + 1];
    const int64_t r = (int64_t)blockIdx.x * kSkyThreads + threadIdx.x;
    const bool live = r < total;
    const int k = live ? find_seg(seg_off, nseg, r) : 0;
    const int64_t s0 = live ? seg_off[k] : 0;
    const uint32_t delta = live ? seg_delta[k] : 0u;
    uint32_t pv[kMaxD];
    const uint32_t jp = live ? items[perm[r]] : 0u;
#pragma unroll
    for (int i = 0; i < kMaxD; i++) pv[i] = (live && i < d) ? p_ord[(int64_t)jp * d + i] : 0u;
    // the block scans [min s0 of its items, its last item)
    const int64_t r_first = (int64_t)blockIdx.x * kSkyThreads;
    __shared__ int64_t s_lo;
    if (threadIdx.x == 0) s_lo = seg_off[find_seg(seg_off, nseg, r_first)];
    __syncthreads();
    const int64_t lo = s_lo, hi = min(total, r_first + kSkyThreads);
    int st = 0;  // 0 undominated, 1 dominated, 2 strictly dominated
    for (int64_t t0 = lo; t0 < hi; t0 += kSkyThreads) {
        const int64_t q = t0 + threadIdx.x;
        if (q < hi) {
            const uint32_t jq = items[perm[q]];
            for (int i = 0; i < d; i++) tile[threadIdx.x][i] = p_ord[(int64_t)jq * d + i];
        }
        __syncthreads();
        if (live && st < 2) {
            const int64_t qa = max(t0, s0), qb = min(t0 + kSkyThreads, r);
            for (int64_t qq = qa; qq < qb; qq++) {
                const uint32_t *qv = tile[qq - t0];
                bool le = true, lt_any = false, lt_all = true;
                for (int i = 0; i < d; i++) {
                    if (!((delta >> i) & 1u)) continue;
                    const uint32_t a = qv[i], b = pv[i];
                    le &= a <= b;
                    lt_any |= a < b;
                    lt_all &= a < b;
                }
                if (lt_all) {
                    st = 2;
                    break;
                }
                if (le && lt_any) st = 1;
            }
        }
        if (__syncthreads_and(!live || st == 2)) break;  // every item of the block is settled
    }
    if (live) status[perm[r]] = (uint8_t)st;  // back to the input (ascending j) order
}

// flags for the compaction: keep = status <= 1 (in S+_delta), sky = status == 0 (in S_delta)
__global__ void sdsc_flags_kernel(const uint8_t *__restrict__ status, int64_t total, uint32_t *__restrict__ keep,
                                  uint32_t *__restrict__ sky) {
    const int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (e >= total) return;
    keep[e] = status[e] <= 1 ? 1u : 0u;
    sky[e] = status[e] == 0 ? 1u : 0u;
}

// next level's lists: item j with bit 31 = in S_delta; per-segment counts via the scans at segment ends
__global__ void sdsc_compact_kernel(const uint32_t *__restrict__ items, const uint8_t *__restrict__ status,
                                    const uint32_t *__restrict__ keep_idx, int64_t total, uint32_t *__restrict__ out) {
    const int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (e >= total || status[e] > 1) return;
    out[keep_idx[e]] = items[e] | (status[e] == 0 ? 0x80000000u : 0u);
}

__global__ void sdsc_seg_counts_kernel(const uint32_t *__restrict__ keep, const uint32_t *__restrict__ keep_idx,
                                       const uint32_t *__restrict__ sky, const uint32_t *__restrict__ sky_idx,
                                       const int64_t *__restrict__ seg_off, int nseg, int64_t *__restrict__ cnt) {
    const int k = blockIdx.x * blockDim.x + threadIdx.x;
    if (k >= nseg) return;
    const int64_t a = seg_off[k], b = seg_off[k + 1];
    int64_t ka = 0, kb = 0, sa = 0, sb = 0;
    if (b > a) {
        ka = keep_idx[a];
        kb = keep_idx[b - 1] + keep[b - 1];
        sa = sky_idx[a];
        sb = sky_idx[b - 1] + sky[b - 1];
    }
    cnt[2 * k] = kb - ka;      // |S+_delta| (= |L| + |L+|)
    cnt[2 * k + 1] = sb - sa;  // |S_delta|
    (void)ka;
}

// the level's S_delta ids into the output lattice: ids[lat_off[k] + rank] = ext_ids[j]
__global__ void sdsc_emit_kernel(const uint32_t *__restrict__ items, const uint32_t *__restrict__ sky,
                                 const uint32_t *__restrict__ sky_idx, const int64_t *__restrict__ seg_off,
                                 const int64_t *__restrict__ lat_off, int nseg, int64_t total,
                                 const int32_t *__restrict__ ext_ids, int32_t *__restrict__ ids) {
    const int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (e >= total || !sky[e]) return;
    const int k = find_seg(seg_off, nseg, e);
    const int64_t rank = (int64_t)sky_idx[e] - (int64_t)sky_idx[seg_off[k]];
    ids[lat_off[k] + rank] = ext_ids[items[e]];
}

// final lattice assembly: block b copies subspace b's ids from the level staging area (one launch, instead
// of one copy call per subspace)
__global__ void sdsc_assemble_kernel(const int64_t *__restrict__ src, const int64_t *__restrict__ dst,
                                     const int64_t *__restrict__ len, const int32_t *__restrict__ staging,
                                     int32_t *__restrict__ ids) {
    const int64_t b = blockIdx.x;
    const int64_t s = src[b], t = dst[b], l = len[b];
    for (int64_t i = threadIdx.x; i < l; i += blockDim.x) ids[t + i] = staging[s + i];
}

// membership rows from the lattice: bit delta of row id for every (delta, id)
__global__ void sdsc_rows_kernel(const int64_t *__restrict__ offsets, int64_t nsub, const int32_t *__restrict__ ids,
                                 int64_t total, uint32_t W, uint32_t *__restrict__ membership) {
    const int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (e >= total) return;
    int64_t lo = 0, hi = nsub;  // offsets[lo] <= e < offsets[hi]
    while (hi - lo > 1) {
        const int64_t mid = (lo + hi) >> 1;
        if (offsets[mid] <= e) lo = mid;
        else hi = mid;
    }
    atomicOr(&membership[(int64_t)ids[e] * W + (lo >> 5)], 1u << (lo & 31));
}

unsigned blocks(int64_t n, int t) { return (unsigned)ceil_div(n > 0 ? n : 1, t); }

int bitlen(uint64_t x) {
    int b = 0;
    while (x) {
        b++;
        x >>= 1;
    }
    return b;
}

}  // namespace

// Alg. 2 over the installed S+(P) (after prep + prefilter + ext_build).  Writes the lattice into the device
// buffers d_offsets[2^d+1] / *d_ids (allocated here in c.sdsc_ids) and the membership rows into d_membership
// [n*W] (nullable).  Returns the total number of ids.  Host-orchestrated: one batched pass per level.
int64_t sdsc_run(Ctx &c, int64_t *d_offsets, uint32_t *d_membership, cudaStream_t st, int32_t **d_ids_out) {
    if (!c.ext_ready) throw Error{1, "SDSC before the extended skyline is installed"};
    const int d = c.d;
    const int64_t m = c.m;
    const int64_t nsub = (int64_t)1 << d;
    const uint32_t full = (uint32_t)(nsub - 1);
    std::vector<int64_t> plus_cnt(nsub, 0), sky_cnt(nsub, 0), list_off(nsub, -1);
    std::vector<uint32_t> level_deltas;
    // lists of the previous level (device), indexed by list_off[delta]
    DevBuf &prev = c.sdsc_prev, &next = c.sdsc_next;
    // level-by-level the emitted S_delta go to a staging area; final lattice assembled at the end
    std::vector<int64_t> lat_len(nsub, 0);
    std::vector<std::pair<uint32_t, int64_t>> emitted;  // (delta, offset into c.sdsc_ids_tmp)
    int64_t emitted_total = 0;
    DevBuf &ids_tmp = c.sdsc_ids_tmp;
    for (int level = d; level >= 1; level--) {
        level_deltas.clear();
        for (uint32_t delta = 1; delta <= full; delta++)
            if (__builtin_popcount(delta) == level) level_deltas.push_back(delta);
        const int nseg = (int)level_deltas.size();
        std::vector<int64_t> seg_off(nseg + 1, 0), src_off(nseg, 0);
        for (int k = 0; k < nseg; k++) {
            const uint32_t delta = level_deltas[k];
            int64_t len;
            if (level == d) {
                len = m;
            } else {
                uint32_t parent = 0;
                int64_t best = -1;
                for (int i = 0; i < d; i++) {  // Alg. 2 line 5 (reading S1: smallest size, then smallest delta')
                    if ((delta >> i) & 1u) continue;
                    const uint32_t p = delta | (1u << i);
                    if (best < 0 || plus_cnt[p] < best || (plus_cnt[p] == best && p < parent)) {
                        best = plus_cnt[p];
                        parent = p;
                    }
                }
                len = best;
                src_off[k] = list_off[parent];
            }
            seg_off[k + 1] = seg_off[k] + len;
        }
        const int64_t total = seg_off[nseg];
        // device tables
        c.sdsc_tab.ensure(sizeof(int64_t) * (2 * (size_t)nseg + 4) + sizeof(uint32_t) * (size_t)nseg + 64);
        int64_t *d_seg_off = c.sdsc_tab.as<int64_t>();
        int64_t *d_src_off = d_seg_off + nseg + 1;
        uint32_t *d_seg_delta = reinterpret_cast<uint32_t *>(d_src_off + nseg + 1);
        SKY_CUDA(cudaMemcpyAsync(d_seg_off, seg_off.data(), sizeof(int64_t) * (nseg + 1), cudaMemcpyHostToDevice, st));
        SKY_CUDA(cudaMemcpyAsync(d_src_off, src_off.data(), sizeof(int64_t) * nseg, cudaMemcpyHostToDevice, st));
        SKY_CUDA(cudaMemcpyAsync(d_seg_delta, level_deltas.data(), sizeof(uint32_t) * nseg, cudaMemcpyHostToDevice, st));
        std::vector<int64_t> cnt(2 * (size_t)nseg, 0);
        if (total > 0) {
            c.sdsc_items.ensure(sizeof(uint32_t) * total);
            c.sdsc_keys.ensure(sizeof(uint64_t) * total);
            c.sdsc_vals.ensure(sizeof(uint32_t) * total);
            c.sdsc_keys_alt.ensure(sizeof(uint64_t) * total);
            c.sdsc_vals_alt.ensure(sizeof(uint32_t) * total);
            c.sdsc_counts.ensure(sizeof(uint32_t) * radix_scratch_counts(total));
            c.sdsc_scan.ensure(scan_tmp_bytes(std::max<int64_t>((int64_t)radix_scratch_counts(total), total)));
            c.sdsc_status.ensure(total);
            c.sdsc_flags.ensure(sizeof(uint32_t) * 4 * (size_t)total);
            uint32_t *items = c.sdsc_items.as<uint32_t>();
            sdsc_gather_kernel<<<(unsigned)std::min<int64_t>(blocks(total, 256), (int64_t)c.num_sms * 32), 256, 0, st>>>(
                level == d ? nullptr : prev.as<uint32_t>(), d_src_off, d_seg_off, d_seg_delta, nseg, total,
                c.p_ord.as<uint32_t>(), d, items, c.sdsc_keys.as<uint64_t>(), c.sdsc_vals.as<uint32_t>());
            c.L.count++;
            SKY_LAUNCH_CHECK();
            radix_sort_u64(c.sdsc_keys.as<uint64_t>(), c.sdsc_vals.as<uint32_t>(), total, 36 + bitlen((uint64_t)nseg),
                           c.sdsc_keys_alt.as<uint64_t>(), c.sdsc_vals_alt.as<uint32_t>(), c.sdsc_counts.as<uint32_t>(),
                           c.sdsc_scan.p, st, c.L);
            uint8_t *status = c.sdsc_status.as<uint8_t>();
            sdsc_sky_kernel<<<blocks(total, kSkyThreads), kSkyThreads, 0, st>>>(
                items, c.sdsc_vals.as<uint32_t>(), d_seg_off, d_seg_delta, nseg, total, c.p_ord.as<uint32_t>(), d, status);
            c.L.count++;
            SKY_LAUNCH_CHECK();
            uint32_t *keep = c.sdsc_flags.as<uint32_t>(), *keep_idx = keep + total, *sky = keep_idx + total,
                     *sky_idx = sky + total;
            sdsc_flags_kernel<<<blocks(total, 256), 256, 0, st>>>(status, total, keep, sky);
            c.L.count++;
            SKY_LAUNCH_CHECK();
            exclusive_scan_u32(keep, keep_idx, total, c.sdsc_scan.p, st, c.L);
            exclusive_scan_u32(sky, sky_idx, total, c.sdsc_scan.p, st, c.L);
            c.sdsc_cnt.ensure(sizeof(int64_t) * 2 * (size_t)nseg);
            sdsc_seg_counts_kernel<<<blocks(nseg, 128), 128, 0, st>>>(keep, keep_idx, sky, sky_idx, d_seg_off, nseg,
                                                                     c.sdsc_cnt.as<int64_t>());
            c.L.count++;
            SKY_LAUNCH_CHECK();
            SKY_CUDA(cudaMemcpyAsync(cnt.data(), c.sdsc_cnt.p, sizeof(int64_t) * 2 * nseg, cudaMemcpyDeviceToHost, st));
            SKY_CUDA(cudaStreamSynchronize(st));
            int64_t kept = 0, skyt = 0;
            for (int k = 0; k < nseg; k++) {
                kept += cnt[2 * k];
                skyt += cnt[2 * k + 1];
            }
            next.ensure(sizeof(uint32_t) * (size_t)std::max<int64_t>(kept, 1));
            sdsc_compact_kernel<<<blocks(total, 256), 256, 0, st>>>(items, status, keep_idx, total, next.as<uint32_t>());
            c.L.count++;
            SKY_LAUNCH_CHECK();
            // S_delta of this level -> staging (grow-only, copy on growth)
            if (skyt > 0) {
                const size_t need = sizeof(int32_t) * (size_t)(emitted_total + skyt);
                if (need > ids_tmp.bytes) {
                    DevBuf bigger;
                    bigger.ensure(need * 2);
                    if (emitted_total)
                        SKY_CUDA(cudaMemcpyAsync(bigger.p, ids_tmp.p, sizeof(int32_t) * emitted_total,
                                                 cudaMemcpyDeviceToDevice, st));
                    SKY_CUDA(cudaStreamSynchronize(st));
                    ids_tmp.release();
                    ids_tmp = bigger;
                    bigger.p = nullptr;
                    bigger.bytes = 0;
                }
                std::vector<int64_t> lat_off(nseg, 0);
                int64_t o = emitted_total;
                for (int k = 0; k < nseg; k++) {
                    lat_off[k] = o;
                    o += cnt[2 * k + 1];
                }
                c.sdsc_lat.ensure(sizeof(int64_t) * (size_t)nseg);
                SKY_CUDA(cudaMemcpyAsync(c.sdsc_lat.p, lat_off.data(), sizeof(int64_t) * nseg, cudaMemcpyHostToDevice, st));
                sdsc_emit_kernel<<<blocks(total, 256), 256, 0, st>>>(items, sky, sky_idx, d_seg_off,
                                                                     c.sdsc_lat.as<int64_t>(), nseg, total,
                                                                     c.ext_ids.as<int32_t>(), ids_tmp.as<int32_t>());
                c.L.count++;
                SKY_LAUNCH_CHECK();
                for (int k = 0; k < nseg; k++) emitted.push_back({level_deltas[k], lat_off[k]});
                emitted_total = o;
            } else {
                for (int k = 0; k < nseg; k++) emitted.push_back({level_deltas[k], emitted_total});
            }
            std::swap(prev.p, next.p);
            std::swap(prev.bytes, next.bytes);
        } else {
            for (int k = 0; k < nseg; k++) emitted.push_back({level_deltas[k], emitted_total});
        }
        int64_t o = 0;
        for (int k = 0; k < nseg; k++) {
            const uint32_t delta = level_deltas[k];
            plus_cnt[delta] = cnt[2 * k];
            sky_cnt[delta] = cnt[2 * k + 1];
            list_off[delta] = o;
            o += cnt[2 * k];
        }
    }
    // final lattice: offsets by delta, ids copied from the staging area per delta
    std::vector<int64_t> offsets(nsub + 1, 0);
    for (int64_t delta = 1; delta < nsub; delta++) offsets[delta + 1] = offsets[delta] + sky_cnt[delta];
    offsets[1] = 0;
    const int64_t total_ids = offsets[nsub];
    c.sdsc_ids.ensure(sizeof(int32_t) * (size_t)std::max<int64_t>(total_ids, 1));
    if (total_ids > 0) {
        std::vector<int64_t> tab(3 * emitted.size());
        const size_t ne = emitted.size();
        for (size_t i = 0; i < ne; i++) {
            tab[i] = emitted[i].second;
            tab[ne + i] = offsets[emitted[i].first];
            tab[2 * ne + i] = sky_cnt[emitted[i].first];
        }
        c.sdsc_tab.ensure(sizeof(int64_t) * tab.size());
        SKY_CUDA(cudaMemcpyAsync(c.sdsc_tab.p, tab.data(), sizeof(int64_t) * tab.size(), cudaMemcpyHostToDevice, st));
        const int64_t *t = c.sdsc_tab.as<int64_t>();
        sdsc_assemble_kernel<<<(unsigned)ne, 128, 0, st>>>(t, t + ne, t + 2 * ne, ids_tmp.as<int32_t>(),
                                                           c.sdsc_ids.as<int32_t>());
        c.L.count++;
        SKY_LAUNCH_CHECK();
    }
    SKY_CUDA(cudaMemcpyAsync(d_offsets, offsets.data(), sizeof(int64_t) * (nsub + 1), cudaMemcpyHostToDevice, st));
    if (d_membership) {
        SKY_CUDA(cudaMemsetAsync(d_membership, 0, sizeof(uint32_t) * (size_t)c.n * c.W, st));
        if (total_ids > 0) {
            sdsc_rows_kernel<<<blocks(total_ids, 256), 256, 0, st>>>(d_offsets, nsub, c.sdsc_ids.as<int32_t>(), total_ids,
                                                                   c.W, d_membership);
            c.L.count++;
            SKY_LAUNCH_CHECK();
        }
    }
    SKY_CUDA(cudaStreamSynchronize(st));  // host vectors above feed async copies
    *d_ids_out = c.sdsc_ids.as<int32_t>();
    return total_ids;
}

}  // namespace sky
