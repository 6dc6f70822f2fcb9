// capi.cu — the C-ABI of include/skycube.h: argument validation, the per-device context cache,
// pinned host-memory pool for results, phase orchestration on one stream, and per-phase CUDA-event
// statistics.  Every compute step runs in the kernels of prep.cu / k1_prefilter.cu / k3_mdmc.cu /
// k4_compact.cu; there is no CPU fallback: without an sm_100 device every call fails with ENODEV.
#include <algorithm>
#include <chrono>
#include <cstring>
#include <map>
#include <mutex>
#include <unordered_map>
#include <vector>

#include "../../include/skycube.h"
#include "ctx.cuh"

struct skycube_ctx {
    sky::Ctx c;
    sky::DevBuf input, ext8, rows32, ext_rows32, membership, offsets, ids, flag_stage;
    cudaStream_t side = nullptr;  // non-blocking stream for work that overlaps the main (default) stream
    cudaEvent_t ev_ext = nullptr, ev_side = nullptr;
};

namespace sky {
Tuning &tuning() {
    static Tuning t;
    return t;
}
}  // namespace sky

namespace {

std::mutex g_mutex;                  // serialises skycube_build* (header: "calls are serialised")
thread_local std::string g_last_error;

skycube_status fail(skycube_status s, const std::string &msg) {
    g_last_error = msg;
    return s;
}

// ----------------------------------------------------------------------- pinned host memory pool
struct PinnedPool {
    std::mutex mu;
    std::multimap<size_t, void *> free_;
    std::unordered_map<void *, size_t> size_of;
    size_t cached = 0;
    static constexpr size_t kMaxCached = (size_t)48 << 30;

    void *get(size_t bytes) {
        if (bytes == 0) bytes = 64;
        {
            std::lock_guard<std::mutex> lk(mu);
            auto it = free_.lower_bound(bytes);
            if (it != free_.end() && it->first <= bytes + bytes / 2 + (1 << 20)) {
                void *p = it->second;
                cached -= it->first;
                free_.erase(it);
                return p;
            }
        }
        void *p = nullptr;
        if (cudaMallocHost(&p, bytes) != cudaSuccess) {
            cudaGetLastError();
            // drop the cache and retry once
            release_all();
            if (cudaMallocHost(&p, bytes) != cudaSuccess) {
                cudaGetLastError();
                throw sky::Error{3, "cudaMallocHost(" + std::to_string(bytes) + ") failed"};
            }
        }
        std::lock_guard<std::mutex> lk(mu);
        size_of[p] = bytes;
        return p;
    }
    void put(void *p) {
        if (!p) return;
        std::lock_guard<std::mutex> lk(mu);
        auto it = size_of.find(p);
        if (it == size_of.end()) return;
        if (cached + it->second > kMaxCached) {
            cudaFreeHost(p);
            size_of.erase(it);
            return;
        }
        free_.emplace(it->second, p);
        cached += it->second;
    }
    void release_all() {
        std::lock_guard<std::mutex> lk(mu);
        for (auto &kv : free_) {
            cudaFreeHost(kv.second);
            size_of.erase(kv.second);
        }
        free_.clear();
        cached = 0;
    }
};
PinnedPool g_pool;

std::map<int, skycube_ctx *> g_ctx;  // one cached context per device for skycube_build*
std::map<int, skycube_ctx *> g_mctx; // multi-GPU builds: one context per (rank, device)

void check_device(int device) {
    int count = 0;
    if (cudaGetDeviceCount(&count) != cudaSuccess || count == 0) {
        cudaGetLastError();
        throw sky::Error{SKYCUBE_ENODEV, "no CUDA device visible"};
    }
    if (device < 0 || device >= count) throw sky::Error{SKYCUBE_ENODEV, "device ordinal out of range"};
    // cudaDeviceGetAttribute, not cudaGetDeviceProperties: the latter queries every property and can
    // cost tens of milliseconds per call (it sat inside the e2e timed region)
    int major = 0;
    SKY_CUDA(cudaDeviceGetAttribute(&major, cudaDevAttrComputeCapabilityMajor, device));
    if (major != 10) throw sky::Error{SKYCUBE_ENODEV, "not an sm_100 device (compute capability " + std::to_string(major) + ".x)"};
    SKY_CUDA(cudaSetDevice(device));
}

skycube_ctx *new_ctx(int device) {
    check_device(device);
    auto *x = new skycube_ctx();
    x->c.device = device;
    int sms = 148;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, device);
    x->c.num_sms = sms;
    x->c.counters.ensure(sizeof(unsigned long long) * 8);
    SKY_CUDA(cudaMemset(x->c.counters.p, 0, sizeof(unsigned long long) * 8));
    return x;
}

template <typename F>
skycube_status guarded(F &&f) {
    try {
        f();
        return SKYCUBE_OK;
    } catch (const sky::Error &e) {
        return fail((skycube_status)e.status, e.msg);
    } catch (const std::bad_alloc &) {
        return fail(SKYCUBE_ENOMEM, "host allocation failed");
    } catch (...) {
        return fail(SKYCUBE_ECUDA, "unexpected exception");
    }
}

// K3 work counters (exact DTs = misses, expansions) of a context, for skycube_stats
void read_k3_counters(const sky::Ctx &c, int64_t *exact_dts, int64_t *expansions) {
    int64_t a[8] = {0};
    SKY_CUDA(cudaSetDevice(c.device));
    SKY_CUDA(cudaMemcpy(a, c.counters.p, sizeof(a), cudaMemcpyDeviceToHost));
    *exact_dts = a[4];
    *expansions = a[6];
}

// Failure after kernels may have been queued: wait for every stream of the device before the result's
// pinned buffers go back to the pool (K3 writes the membership rows straight into one of them).
void drain_device(int device) {
    if (cudaSetDevice(device) == cudaSuccess) cudaDeviceSynchronize();
    cudaGetLastError();
}

float ev_ms(cudaEvent_t a, cudaEvent_t b) {
    float ms = 0.f;
    cudaEventElapsedTime(&ms, a, b);
    return ms;
}

// H2D of the points, then K0/K2 prepare, K1 prefilter, S+ install and K3 MDMC into x->rows32 (tiled
// rows of the S+ points).  Events: ev[0] before H2D, ev[1] after H2D, ev[2] after prepare, ev[3] after
// the prefilter, ev[4] after MDMC.
void device_rows(skycube_ctx *x, const float *points, int64_t n, int d, int max_level, bool want_ext,
                 cudaStream_t s, cudaEvent_t *ev, uint32_t *host_mem = nullptr) {
    sky::Ctx &c = x->c;
    const uint32_t W = sky::words_per_row(d);
    x->input.ensure(sizeof(float) * n * d);
    SKY_CUDA(cudaEventRecord(ev[0], s));
    SKY_CUDA(cudaMemcpyAsync(x->input.p, points, sizeof(float) * n * d, cudaMemcpyHostToDevice, s));
    SKY_CUDA(cudaEventRecord(ev[1], s));
    sky::prep_run(c, x->input.as<float>(), n, d, s);
    SKY_CUDA(cudaEventRecord(ev[2], s));
    x->ext8.ensure(n);
    sky::prefilter_run(c, 0, 1, x->ext8.as<uint8_t>(), s);
    sky::ext_build(c, x->ext8.as<uint8_t>(), s);
    SKY_CUDA(cudaEventRecord(ev[3], s));
    const int64_t m = c.m;
    const size_t rows_words = (size_t)sky::ceil_div(m > 0 ? m : 1, 32) * 32 * W;
    x->rows32.ensure(sizeof(uint32_t) * rows_words);
    if (want_ext) x->ext_rows32.ensure(sizeof(uint32_t) * rows_words);
    c.max_level = max_level;
    if (host_mem) {
        // zero-copy membership: the rows of points outside S+ are zeroed in the pinned host array on a side
        // stream while K3 runs (and writes the S+ rows there itself); the caller joins x->ev_side
        if (!x->side) {
            SKY_CUDA(cudaStreamCreateWithFlags(&x->side, cudaStreamNonBlocking));
            SKY_CUDA(cudaEventCreateWithFlags(&x->ev_ext, cudaEventDisableTiming));
            SKY_CUDA(cudaEventCreateWithFlags(&x->ev_side, cudaEventDisableTiming));
        }
        SKY_CUDA(cudaEventRecord(x->ev_ext, s));
        SKY_CUDA(cudaStreamWaitEvent(x->side, x->ev_ext, 0));
        sky::membership_zero_outside(c, host_mem, x->side);
        SKY_CUDA(cudaEventRecord(x->ev_side, x->side));
    }
    sky::mdmc_run(c, 0, m, x->rows32.as<uint32_t>(), want_ext ? x->ext_rows32.as<uint32_t>() : nullptr, s, host_mem);
    SKY_CUDA(cudaEventRecord(ev[4], s));
}

struct Events {
    cudaEvent_t e[9];
    Events() {
        for (auto &v : e) SKY_CUDA(cudaEventCreate(&v));
    }
    ~Events() {
        for (auto &v : e) cudaEventDestroy(v);
    }
};


// Contiguous task range of shard g of k: 32-task groups split as evenly as possible, in shard order.
inline void shard_range(int64_t m, int k, int g, int64_t *j0, int64_t *j1) {
    const int64_t groups = sky::ceil_div(m, 32);
    const int64_t g0 = groups * g / k, g1 = groups * (g + 1) / k;
    *j0 = std::min<int64_t>(m, g0 * 32);
    *j1 = std::min<int64_t>(m, g1 * 32);
}

// Single-process multi-GPU build: num_gpus = k logical ranks on devices first..first+k-1
// (skycube_set_tuning("share_devices", 1) lets ranks share devices round-robin -- the k-rank logic on one GPU).
//   every rank: H2D of the points, K0/K2 prepare (replicated, deterministic)
//   rank g:     K1 on the prefilter blocks b = g (mod k); the k flag vectors are gathered on rank 0 by peer
//               copies (NVLink), OR-combined and broadcast back; every rank installs S+
//   rank g:     K3 on its contiguous range of 32-task groups; its membership rows go straight into the pinned
//               host result by id (zero-copy over its own PCIe link), and it zeroes the rows of the points
//               outside S+ in its slice of ids
//   rank g:     K4 count pass over its own rows -> per-subspace totals; the k total vectors are exchanged by peer
//               copies (k * 2^d int64); each rank places and writes its own ids straight into the pinned host
//               lattice at their global positions
// Nothing of size n or of the lattice crosses between GPUs; the output bytes equal the single-GPU build's.
skycube_status build_multi(const float *points, int64_t n, int d, int first, int k, int max_level, bool lists,
                           skycube_result *out, skycube_stats *stats) {
    std::lock_guard<std::mutex> lk(g_mutex);
    const auto t0 = std::chrono::steady_clock::now();
    skycube_result r;
    std::memset(&r, 0, sizeof(r));
    skycube_status st = guarded([&] {
        int count = 0;
        if (cudaGetDeviceCount(&count) != cudaSuccess || count == 0) {
            cudaGetLastError();
            throw sky::Error{SKYCUBE_ENODEV, "no CUDA device visible"};
        }
        const bool share = sky::tuning().share_devices == 1;
        if (!share && first + k > count)
            throw sky::Error{SKYCUBE_ENODEV, "num_gpus exceeds the visible devices after `device`"};
        std::vector<int> dev(k);
        std::vector<skycube_ctx *> xs(k);
        for (int g = 0; g < k; g++) {
            dev[g] = (first + g) % count;
            check_device(dev[g]);
            skycube_ctx *&x = g_mctx[(g << 8) | dev[g]];
            if (!x) x = new_ctx(dev[g]);
            xs[g] = x;
        }
        for (int g = 0; g < k; g++)  // NVLink peer access between every pair of distinct devices
            for (int h = 0; h < k; h++) {
                if (dev[g] == dev[h]) continue;
                int can = 0;
                cudaDeviceCanAccessPeer(&can, dev[g], dev[h]);
                if (can) {
                    SKY_CUDA(cudaSetDevice(dev[g]));
                    if (cudaDeviceEnablePeerAccess(dev[h], 0) != cudaSuccess) cudaGetLastError();
                }
            }
        r.d = d;
        r.n = n;
        r.words_per_row = sky::words_per_row(d);
        const uint32_t W = r.words_per_row;
        const int64_t nsub = (int64_t)1 << d;
        auto sync_all = [&] {
            for (int g = 0; g < k; g++) {
                SKY_CUDA(cudaSetDevice(dev[g]));
                SKY_CUDA(cudaDeviceSynchronize());
            }
        };
        using clk = std::chrono::steady_clock;
        double ms_comm = 0;
        auto ms = [](clk::time_point a, clk::time_point b) { return std::chrono::duration<double, std::milli>(b - a).count(); };
        int64_t launches0 = 0, dts0 = 0, exp0 = 0;
        for (int g = 0; g < k; g++) {
            launches0 += xs[g]->c.L.count;
            if (stats) {
                int64_t a = 0, b = 0;
                read_k3_counters(xs[g]->c, &a, &b);
                dts0 += a;
                exp0 += b;
            }
        }
        const auto tp0 = clk::now();
        // prepare (replicated) + the rank's prefilter blocks
        for (int g = 0; g < k; g++) {
            skycube_ctx *x = xs[g];
            SKY_CUDA(cudaSetDevice(dev[g]));
            x->input.ensure(sizeof(float) * n * d);
            SKY_CUDA(cudaMemcpyAsync(x->input.p, points, sizeof(float) * n * d, cudaMemcpyHostToDevice, nullptr));
            sky::prep_run(x->c, x->input.as<float>(), n, d, nullptr);
            x->ext8.ensure(n);
            SKY_CUDA(cudaMemsetAsync(x->ext8.p, 0, n, nullptr));
            sky::prefilter_run(x->c, g, k, x->ext8.as<uint8_t>(), nullptr);
        }
        sync_all();
        // exchange 1: gather the flags on rank 0, OR, broadcast
        const auto tc0 = clk::now();
        skycube_ctx *x0 = xs[0];
        SKY_CUDA(cudaSetDevice(dev[0]));
        x0->flag_stage.ensure((size_t)n * k);
        for (int g = 0; g < k; g++)
            SKY_CUDA(cudaMemcpyPeerAsync(x0->flag_stage.as<uint8_t>() + (size_t)g * n, dev[0], xs[g]->ext8.p, dev[g], n, nullptr));
        sky::or_flags(x0->c, x0->flag_stage.as<uint8_t>(), k, n, x0->ext8.as<uint8_t>(), nullptr);
        for (int g = 1; g < k; g++)
            SKY_CUDA(cudaMemcpyPeerAsync(xs[g]->ext8.p, dev[g], x0->ext8.p, dev[0], n, nullptr));
        sync_all();
        ms_comm += ms(tc0, clk::now());
        const auto tp1 = clk::now();
        for (int g = 0; g < k; g++) {
            SKY_CUDA(cudaSetDevice(dev[g]));
            sky::ext_build(xs[g]->c, xs[g]->ext8.as<uint8_t>(), nullptr);
        }
        const int64_t m = x0->c.m;
        const size_t rows_words = (size_t)std::max<int64_t>(sky::ceil_div(m, 32), 1) * W * 32;
        r.n_ext = m;
        r.ext_ids = (int32_t *)g_pool.get(sizeof(int32_t) * (m > 0 ? m : 1));
        r.membership = (uint32_t *)g_pool.get(sizeof(uint32_t) * (size_t)n * W);
        std::vector<int64_t> j0(k), j1(k);
        for (int g = 0; g < k; g++) {
            skycube_ctx *x = xs[g];
            SKY_CUDA(cudaSetDevice(dev[g]));
            shard_range(m, k, g, &j0[g], &j1[g]);
            x->rows32.ensure(sizeof(uint32_t) * rows_words);
            x->c.max_level = max_level;
            // K3 writes the rank's rows into the pinned result by id (zero-copy); the rank then zeroes the rows of
            // the points outside S+ in its slice of ids
            if (j1[g] > j0[g]) sky::mdmc_run(x->c, j0[g], j1[g], x->rows32.as<uint32_t>(), nullptr, nullptr, r.membership);
            sky::compact_membership_shard(x->c, x->rows32.as<uint32_t>(), j0[g], j0[g], n * g / k, n * (g + 1) / k,
                                          r.membership, nullptr);
            if (lists) {
                x->offsets.ensure(sizeof(int64_t) * (nsub + 1) + sizeof(int64_t) * (size_t)k * nsub);
                sky::lattice_count_shard(x->c, x->rows32.as<uint32_t>(), j0[g], j1[g],
                                         x->offsets.as<int64_t>() + (nsub + 1) + (size_t)g * nsub, nullptr);
            }
        }
        if (m) {
            SKY_CUDA(cudaSetDevice(dev[0]));
            SKY_CUDA(cudaMemcpyAsync(r.ext_ids, x0->c.ext_ids.p, sizeof(int32_t) * m, cudaMemcpyDeviceToHost, nullptr));
        }
        sync_all();
        const auto tp2 = clk::now();
        int64_t total = 0;
        if (lists) {
            // exchange 2: every rank's per-subspace totals to every rank (k * 2^d int64 by peer copies)
            const auto tc1 = clk::now();
            const size_t tb = sizeof(int64_t) * (size_t)nsub;
            for (int g = 0; g < k; g++) {
                SKY_CUDA(cudaSetDevice(dev[g]));
                int64_t *all_g = xs[g]->offsets.as<int64_t>() + (nsub + 1);
                for (int h = 0; h < k; h++)
                    if (h != g)
                        SKY_CUDA(cudaMemcpyPeerAsync(all_g + (size_t)h * nsub, dev[g],
                                                     xs[h]->offsets.as<int64_t>() + (nsub + 1) + (size_t)h * nsub, dev[h],
                                                     tb, nullptr));
            }
            sync_all();
            ms_comm += ms(tc1, clk::now());
            // the id count (to size the pinned lattice) from rank 0's placement pass, then every rank writes its
            // own segments straight into the pinned host lattice
            SKY_CUDA(cudaSetDevice(dev[0]));
            total = sky::lattice_scatter_shard(x0->c, x0->rows32.as<uint32_t>(), j0[0], j1[0],
                                               x0->offsets.as<int64_t>() + (nsub + 1), k, 0, x0->offsets.as<int64_t>(),
                                               nullptr, nullptr);
            r.cuboid_offsets = (int64_t *)g_pool.get(sizeof(int64_t) * (nsub + 1));
            r.cuboid_ids = (int32_t *)g_pool.get(sizeof(int32_t) * (total > 0 ? total : 1));
            SKY_CUDA(cudaMemcpyAsync(r.cuboid_offsets, x0->offsets.p, sizeof(int64_t) * (nsub + 1), cudaMemcpyDeviceToHost,
                                     nullptr));
            for (int g = 0; g < k; g++) {
                skycube_ctx *x = xs[g];
                SKY_CUDA(cudaSetDevice(dev[g]));
                if (j1[g] > j0[g])
                    sky::lattice_scatter_shard(x->c, x->rows32.as<uint32_t>(), j0[g], j1[g],
                                               x->offsets.as<int64_t>() + (nsub + 1), k, g, nullptr, r.cuboid_ids, nullptr);
            }
        }
        sync_all();
        for (int g = 0; g < k; g++) {
            SKY_CUDA(cudaSetDevice(dev[g]));
            SKY_CUDA(cudaGetLastError());
        }
        const auto tp3 = clk::now();
        if (stats) {  // host clock per phase (several devices)
            stats->ms_sort = ms(tp0, tp1);     // H2D + prepare + prefilter + flag exchange
            stats->ms_mdmc = ms(tp1, tp2);     // S+ install + K3 (rows zero-copy to the host) + K4 counts
            stats->ms_compact = ms(tp2, tp3);  // totals exchange + K4 placement and scatter (ids zero-copy)
            stats->ms_comm = ms_comm;
            stats->n_ext = m;
            stats->pairs = m * (m > 0 ? m - 1 : 0);
            stats->total_ids = total;
            int64_t launches = 0, dts = 0, exps = 0;
            for (int g = 0; g < k; g++) {
                launches += xs[g]->c.L.count;
                int64_t a = 0, b = 0;
                read_k3_counters(xs[g]->c, &a, &b);
                dts += a;
                exps += b;
            }
            stats->kernel_launches = (int32_t)(launches - launches0);
            stats->exact_dts = dts - dts0;
            stats->expansions = exps - exp0;
            stats->num_gpus = k;
        }
    });
    if (st != SKYCUBE_OK) {
        int count = 0;
        if (cudaGetDeviceCount(&count) != cudaSuccess) count = 0;
        for (int g = 0; g < k && count > 0; g++) drain_device((first + g) % count);
        skycube_free(&r);
        return st;
    }
    if (stats)
        stats->ms_total = std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
    *out = r;
    return SKYCUBE_OK;
}

}  // namespace

extern "C" {

const char *skycube_strerror(skycube_status s) {
    switch (s) {
        case SKYCUBE_OK: return "ok";
        case SKYCUBE_EINVAL: return "invalid argument";
        case SKYCUBE_ENAN: return "NaN in input";
        case SKYCUBE_ENOMEM: return "out of memory";
        case SKYCUBE_ECUDA: return "CUDA error";
        case SKYCUBE_ENCCL: return "collective error";
        case SKYCUBE_ENODEV: return "no sm_100 device";
    }
    return "unknown status";
}

const char *skycube_last_error(void) { return g_last_error.c_str(); }

skycube_status skycube_set_tuning(const char *key, int32_t value) {
    if (!key) return fail(SKYCUBE_EINVAL, "key == NULL");
    std::lock_guard<std::mutex> lk(g_mutex);
    sky::Tuning &t = sky::tuning();
    const std::string k(key);
    if (k == "k3_design") {
        if (value != 0 && value != 'A' && value != 'O') return fail(SKYCUBE_EINVAL, "k3_design must be 0, 'A' or 'O'");
        t.k3_design = value;
    } else if (k == "k3_tpc") {
        if (value < 0) return fail(SKYCUBE_EINVAL, "k3_tpc must be >= 0");
        t.k3_tpc = value;
    } else if (k == "k3_warps") {
        if (value != 0 && value != 16 && value != 24) return fail(SKYCUBE_EINVAL, "k3_warps must be 0, 16 or 24");
        t.k3_warps = value;
    } else if (k == "k3_mode") {
        if (value < -1 || value > 2) return fail(SKYCUBE_EINVAL, "k3_mode must be in [-1, 2]");
        t.k3_mode = value;
    } else if (k == "share_devices") {
        t.share_devices = value ? 1 : 0;
    } else if (k == "reset") {
        t = sky::Tuning();
    } else {
        return fail(SKYCUBE_EINVAL, "unknown tuning key " + k);
    }
    return SKYCUBE_OK;
}

void skycube_free(skycube_result *out) {
    if (!out) return;
    g_pool.put(out->ext_ids);
    g_pool.put(out->membership);
    g_pool.put(out->ext_membership);
    g_pool.put(out->cuboid_offsets);
    g_pool.put(out->cuboid_ids);
    std::memset(out, 0, sizeof(*out));
}

skycube_status skycube_build_ex(const float *points, int64_t n, int32_t d, const skycube_opts *opts,
                                skycube_result *out, skycube_stats *stats) {
    if (!out) return fail(SKYCUBE_EINVAL, "out == NULL");
    std::memset(out, 0, sizeof(*out));
    if (stats) std::memset(stats, 0, sizeof(*stats));
    if (d < 1 || d > 16) return fail(SKYCUBE_EINVAL, "d must be in [1, 16]");
    if (n < 0 || n > INT32_MAX) return fail(SKYCUBE_EINVAL, "n must be in [0, INT32_MAX]");
    if (n > 0 && !points) return fail(SKYCUBE_EINVAL, "points == NULL");
    const uint32_t flags = opts ? opts->flags : 0u;
    const int device = opts ? opts->device : 0;
    const int max_level = opts ? opts->max_level : 0;
    if (max_level < 0 || max_level > d) return fail(SKYCUBE_EINVAL, "max_level must be in [0, d]");
    const int num_gpus = opts ? opts->num_gpus : 1;
    if (num_gpus < 0 || num_gpus > 64) return fail(SKYCUBE_EINVAL, "num_gpus must be in [0, 64]");
    if (num_gpus > 1 && n > 0) {
        if (flags & SKYCUBE_EXT_MEMBERSHIP) return fail(SKYCUBE_EINVAL, "EXT_MEMBERSHIP is single-GPU only");
        return build_multi(points, n, d, device, num_gpus, max_level, !(flags & SKYCUBE_NO_LISTS), out, stats);
    }
    std::lock_guard<std::mutex> lk(g_mutex);
    const auto t0 = std::chrono::steady_clock::now();
    skycube_result r;
    std::memset(&r, 0, sizeof(r));
    skycube_status st = guarded([&] {
        r.d = d;
        r.n = n;
        r.words_per_row = sky::words_per_row(d);
        const uint32_t W = r.words_per_row;
        const int64_t nsub = (int64_t)1 << d;
        skycube_ctx *&x = g_ctx[device];
        if (!x) x = new_ctx(device);
        else check_device(device);
        sky::Ctx &c = x->c;
        const int64_t launches0 = c.L.count;
        int64_t dts0 = 0, exp0 = 0;
        if (stats) read_k3_counters(c, &dts0, &exp0);
        const bool want_ext = (flags & SKYCUBE_EXT_MEMBERSHIP) != 0;
        if (n == 0) {
            if (!(flags & SKYCUBE_NO_LISTS)) {
                r.cuboid_offsets = (int64_t *)g_pool.get(sizeof(int64_t) * (nsub + 1));
                std::memset(r.cuboid_offsets, 0, sizeof(int64_t) * (nsub + 1));
            }
            return;
        }
        cudaStream_t s = nullptr;
        Events evs;
        cudaEvent_t *ev = evs.e;
        // membership goes to the pinned result buffer by zero-copy from K3 (unless the debug ext rows are
        // requested: then the device transpose + copy path below)
        r.membership = (uint32_t *)g_pool.get(sizeof(uint32_t) * (size_t)n * W);
        uint32_t *host_mem = want_ext ? nullptr : r.membership;
        device_rows(x, points, n, d, max_level, want_ext, s, ev, host_mem);
        const int64_t m = c.m;
        if (!host_mem) {
            x->membership.ensure(sizeof(uint32_t) * (size_t)n * W);
            sky::compact_membership(c, x->rows32.as<uint32_t>(), x->membership.as<uint32_t>(), s);
        }
        int64_t total = 0;
        const bool lists = !(flags & SKYCUBE_NO_LISTS);
        if (lists) {
            x->offsets.ensure(sizeof(int64_t) * (nsub + 1));
            sky::compact_lattice(c, x->rows32.as<uint32_t>(), x->offsets.as<int64_t>(), nullptr, &total, s);
            x->ids.ensure(sizeof(int32_t) * (total > 0 ? total : 1));
            sky::compact_lattice(c, x->rows32.as<uint32_t>(), x->offsets.as<int64_t>(), x->ids.as<int32_t>(), &total, s);
        }
        SKY_CUDA(cudaEventRecord(ev[5], s));
        // device -> pinned host
        r.n_ext = m;
        r.ext_ids = (int32_t *)g_pool.get(sizeof(int32_t) * (m > 0 ? m : 1));
        if (m) SKY_CUDA(cudaMemcpyAsync(r.ext_ids, c.ext_ids.p, sizeof(int32_t) * m, cudaMemcpyDeviceToHost, s));
        if (host_mem) {
            SKY_CUDA(cudaStreamWaitEvent(s, x->ev_side, 0));
        } else {
            SKY_CUDA(cudaMemcpyAsync(r.membership, x->membership.p, sizeof(uint32_t) * (size_t)n * W,
                                     cudaMemcpyDeviceToHost, s));
        }
        if (lists) {
            r.cuboid_offsets = (int64_t *)g_pool.get(sizeof(int64_t) * (nsub + 1));
            r.cuboid_ids = (int32_t *)g_pool.get(sizeof(int32_t) * (total > 0 ? total : 1));
            SKY_CUDA(cudaMemcpyAsync(r.cuboid_offsets, x->offsets.p, sizeof(int64_t) * (nsub + 1),
                                     cudaMemcpyDeviceToHost, s));
            if (total)
                SKY_CUDA(cudaMemcpyAsync(r.cuboid_ids, x->ids.p, sizeof(int32_t) * total, cudaMemcpyDeviceToHost, s));
        }
        if (want_ext) {
            sky::compact_membership(c, x->ext_rows32.as<uint32_t>(), x->membership.as<uint32_t>() , s);
            r.ext_membership = (uint32_t *)g_pool.get(sizeof(uint32_t) * (size_t)n * W);
            SKY_CUDA(cudaMemcpyAsync(r.ext_membership, x->membership.p, sizeof(uint32_t) * (size_t)n * W,
                                     cudaMemcpyDeviceToHost, s));
        }
        SKY_CUDA(cudaEventRecord(ev[6], s));
        SKY_CUDA(cudaStreamSynchronize(s));
        SKY_CUDA(cudaGetLastError());
        if (stats) {
            stats->ms_h2d = ev_ms(ev[0], ev[1]);
            stats->ms_validate = 0;  // K0 + sorts + codes are one phase (prep)
            stats->ms_sort = ev_ms(ev[1], ev[2]);
            stats->ms_codes = 0;
            stats->ms_prefilter = ev_ms(ev[2], ev[3]);
            stats->ms_mdmc = ev_ms(ev[3], ev[4]);
            stats->ms_compact = ev_ms(ev[4], ev[5]);
            stats->ms_d2h = ev_ms(ev[5], ev[6]);
            stats->n_ext = m;
            stats->pairs = m * (m > 0 ? m - 1 : 0);
            stats->total_ids = total;
            stats->kernel_launches = (int32_t)(c.L.count - launches0);
            read_k3_counters(c, &stats->exact_dts, &stats->expansions);
            stats->exact_dts -= dts0;
            stats->expansions -= exp0;
            stats->num_gpus = 1;
        }
    });
    if (st != SKYCUBE_OK) {
        drain_device(device);
        skycube_free(&r);
        return st;
    }
    if (stats)
        stats->ms_total = std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
    *out = r;
    return SKYCUBE_OK;
}

skycube_status skycube_build(const float *points, int64_t n, int32_t d, skycube_result *out) {
    return skycube_build_ex(points, n, d, nullptr, out, nullptr);
}

// ------------------------------------------------------------------------------ SDSC comparator (NEXT-3)
skycube_status skycube_build_sdsc(const float *points, int64_t n, int32_t d, const skycube_opts *opts,
                                  skycube_result *out, skycube_stats *stats) {
    if (!out) return fail(SKYCUBE_EINVAL, "out == NULL");
    std::memset(out, 0, sizeof(*out));
    if (stats) std::memset(stats, 0, sizeof(*stats));
    if (d < 1 || d > 16) return fail(SKYCUBE_EINVAL, "d must be in [1, 16]");
    if (n < 0 || n > INT32_MAX) return fail(SKYCUBE_EINVAL, "n must be in [0, INT32_MAX]");
    if (n > 0 && !points) return fail(SKYCUBE_EINVAL, "points == NULL");
    const int device = opts ? opts->device : 0;
    std::lock_guard<std::mutex> lk(g_mutex);
    const auto t0 = std::chrono::steady_clock::now();
    skycube_result r;
    std::memset(&r, 0, sizeof(r));
    skycube_status st = guarded([&] {
        r.d = d;
        r.n = n;
        r.words_per_row = sky::words_per_row(d);
        const uint32_t W = r.words_per_row;
        const int64_t nsub = (int64_t)1 << d;
        skycube_ctx *&x = g_ctx[device];
        if (!x) x = new_ctx(device);
        else check_device(device);
        sky::Ctx &c = x->c;
        const int64_t launches0 = c.L.count;
        r.cuboid_offsets = (int64_t *)g_pool.get(sizeof(int64_t) * (nsub + 1));
        if (n == 0) {
            std::memset(r.cuboid_offsets, 0, sizeof(int64_t) * (nsub + 1));
            return;
        }
        cudaStream_t s = nullptr;
        Events evs;
        cudaEvent_t *ev = evs.e;
        x->input.ensure(sizeof(float) * n * d);
        SKY_CUDA(cudaEventRecord(ev[0], s));
        SKY_CUDA(cudaMemcpyAsync(x->input.p, points, sizeof(float) * n * d, cudaMemcpyHostToDevice, s));
        SKY_CUDA(cudaEventRecord(ev[1], s));
        sky::prep_run(c, x->input.as<float>(), n, d, s);
        SKY_CUDA(cudaEventRecord(ev[2], s));
        x->ext8.ensure(n);
        sky::prefilter_run(c, 0, 1, x->ext8.as<uint8_t>(), s);
        sky::ext_build(c, x->ext8.as<uint8_t>(), s);
        SKY_CUDA(cudaEventRecord(ev[3], s));
        x->offsets.ensure(sizeof(int64_t) * (nsub + 1));
        x->membership.ensure(sizeof(uint32_t) * (size_t)n * W);
        int32_t *d_ids = nullptr;
        const int64_t total = sky::sdsc_run(c, x->offsets.as<int64_t>(), x->membership.as<uint32_t>(), s, &d_ids);
        SKY_CUDA(cudaEventRecord(ev[4], s));
        const int64_t m = c.m;
        r.n_ext = m;
        r.ext_ids = (int32_t *)g_pool.get(sizeof(int32_t) * (m > 0 ? m : 1));
        r.membership = (uint32_t *)g_pool.get(sizeof(uint32_t) * (size_t)n * W);
        r.cuboid_ids = (int32_t *)g_pool.get(sizeof(int32_t) * (total > 0 ? total : 1));
        if (m) SKY_CUDA(cudaMemcpyAsync(r.ext_ids, c.ext_ids.p, sizeof(int32_t) * m, cudaMemcpyDeviceToHost, s));
        SKY_CUDA(cudaMemcpyAsync(r.membership, x->membership.p, sizeof(uint32_t) * (size_t)n * W, cudaMemcpyDeviceToHost, s));
        SKY_CUDA(cudaMemcpyAsync(r.cuboid_offsets, x->offsets.p, sizeof(int64_t) * (nsub + 1), cudaMemcpyDeviceToHost, s));
        if (total) SKY_CUDA(cudaMemcpyAsync(r.cuboid_ids, d_ids, sizeof(int32_t) * total, cudaMemcpyDeviceToHost, s));
        SKY_CUDA(cudaEventRecord(ev[5], s));
        SKY_CUDA(cudaStreamSynchronize(s));
        SKY_CUDA(cudaGetLastError());
        if (stats) {
            stats->ms_h2d = ev_ms(ev[0], ev[1]);
            stats->ms_sort = ev_ms(ev[1], ev[2]);
            stats->ms_prefilter = ev_ms(ev[2], ev[3]);
            stats->ms_mdmc = ev_ms(ev[3], ev[4]);  // the SDSC lattice traversal
            stats->ms_d2h = ev_ms(ev[4], ev[5]);
            stats->n_ext = m;
            stats->pairs = m * (m > 0 ? m - 1 : 0);
            stats->total_ids = total;
            stats->kernel_launches = (int32_t)(c.L.count - launches0);
        }
    });
    if (st != SKYCUBE_OK) {
        drain_device(device);
        skycube_free(&r);
        return st;
    }
    if (stats) {
        stats->num_gpus = 1;
        stats->ms_total = std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
    }
    *out = r;
    return SKYCUBE_OK;
}

// ------------------------------------------------------------------------------ HashCube (NEXT-1/4)
void skycube_hashcube_free(skycube_hashcube *hc) {
    if (!hc) return;
    g_pool.put(hc->word_offsets);
    g_pool.put(hc->keys);
    g_pool.put(hc->key_offsets);
    g_pool.put(hc->ids);
    std::memset(hc, 0, sizeof(*hc));
}

skycube_status skycube_build_hashcube(const float *points, int64_t n, int32_t d, uint32_t w, const skycube_opts *opts,
                                      skycube_hashcube *out, skycube_stats *stats) {
    if (!out) return fail(SKYCUBE_EINVAL, "out == NULL");
    std::memset(out, 0, sizeof(*out));
    if (stats) std::memset(stats, 0, sizeof(*stats));
    if (d < 1 || d > 16) return fail(SKYCUBE_EINVAL, "d must be in [1, 16]");
    if (w < 1 || w > 32) return fail(SKYCUBE_EINVAL, "w must be in [1, 32]");
    if (n < 0 || n > INT32_MAX) return fail(SKYCUBE_EINVAL, "n must be in [0, INT32_MAX]");
    if (n > 0 && !points) return fail(SKYCUBE_EINVAL, "points == NULL");
    const int device = opts ? opts->device : 0;
    const int max_level = opts ? opts->max_level : 0;
    if (max_level < 0 || max_level > d) return fail(SKYCUBE_EINVAL, "max_level must be in [0, d]");
    std::lock_guard<std::mutex> lk(g_mutex);
    const auto t0 = std::chrono::steady_clock::now();
    skycube_hashcube r;
    std::memset(&r, 0, sizeof(r));
    skycube_status st = guarded([&] {
        r.d = d;
        r.w = w;
        r.n = n;
        r.n_words = sky::hashcube_words(d, w);
        skycube_ctx *&x = g_ctx[device];
        if (!x) x = new_ctx(device);
        else check_device(device);
        sky::Ctx &c = x->c;
        const int64_t launches0 = c.L.count;
        if (n == 0) {
            r.word_offsets = (int64_t *)g_pool.get(sizeof(int64_t) * (r.n_words + 1));
            std::memset(r.word_offsets, 0, sizeof(int64_t) * (r.n_words + 1));
            r.key_offsets = (int64_t *)g_pool.get(sizeof(int64_t));
            r.key_offsets[0] = 0;
            return;
        }
        cudaStream_t s = nullptr;
        Events evs;
        cudaEvent_t *ev = evs.e;
        device_rows(x, points, n, d, max_level, false, s, ev);
        sky::hashcube_build(c, x->rows32.as<uint32_t>(), w, s);
        SKY_CUDA(cudaEventRecord(ev[5], s));
        const sky::HashCubeState &h = c.hc;
        r.n_ext = c.m;
        r.total_keys = h.nkeys;
        r.total_ids = h.nvalid;
        r.word_offsets = (int64_t *)g_pool.get(sizeof(int64_t) * (h.nwords + 1));
        r.keys = (uint32_t *)g_pool.get(sizeof(uint32_t) * (h.nkeys > 0 ? h.nkeys : 1));
        r.key_offsets = (int64_t *)g_pool.get(sizeof(int64_t) * (h.nkeys + 1));
        r.ids = (int32_t *)g_pool.get(sizeof(int32_t) * (h.nvalid > 0 ? h.nvalid : 1));
        SKY_CUDA(cudaMemcpyAsync(r.word_offsets, h.woff.p, sizeof(int64_t) * (h.nwords + 1), cudaMemcpyDeviceToHost, s));
        SKY_CUDA(cudaMemcpyAsync(r.key_offsets, h.koff.p, sizeof(int64_t) * (h.nkeys + 1), cudaMemcpyDeviceToHost, s));
        if (h.nkeys) SKY_CUDA(cudaMemcpyAsync(r.keys, h.keys32.p, sizeof(uint32_t) * h.nkeys, cudaMemcpyDeviceToHost, s));
        if (h.nvalid) SKY_CUDA(cudaMemcpyAsync(r.ids, h.vals.p, sizeof(int32_t) * h.nvalid, cudaMemcpyDeviceToHost, s));
        SKY_CUDA(cudaEventRecord(ev[6], s));
        SKY_CUDA(cudaStreamSynchronize(s));
        SKY_CUDA(cudaGetLastError());
        if (stats) {
            stats->ms_h2d = ev_ms(ev[0], ev[1]);
            stats->ms_sort = ev_ms(ev[1], ev[2]);
            stats->ms_prefilter = ev_ms(ev[2], ev[3]);
            stats->ms_mdmc = ev_ms(ev[3], ev[4]);
            stats->ms_compact = ev_ms(ev[4], ev[5]);
            stats->ms_d2h = ev_ms(ev[5], ev[6]);
            stats->n_ext = c.m;
            stats->pairs = c.m * (c.m > 0 ? c.m - 1 : 0);
            stats->total_ids = h.nvalid;
            stats->kernel_launches = (int32_t)(c.L.count - launches0);
        }
    });
    if (st != SKYCUBE_OK) {
        drain_device(device);
        skycube_hashcube_free(&r);
        return st;
    }
    if (stats) stats->num_gpus = 1;
    if (stats)
        stats->ms_total = std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
    *out = r;
    return SKYCUBE_OK;
}

skycube_status skycube_hashcube_query(const skycube_hashcube *hc, uint32_t delta, int32_t *ids, int64_t *count) {
    if (!hc || !count) return fail(SKYCUBE_EINVAL, "NULL argument");
    if (hc->d < 1 || hc->d > 16 || hc->w < 1 || hc->w > 32 || !hc->word_offsets || !hc->key_offsets)
        return fail(SKYCUBE_EINVAL, "not a HashCube built by skycube_build_hashcube");
    if (delta == 0 || delta >= (1u << hc->d)) return fail(SKYCUBE_EINVAL, "delta must be in [1, 2^d - 1]");
    return guarded([&] {
        // L1280 (reading Q6): the lists of h_{(delta-1)/w} whose key has bit (delta-1) % w unset
        const int64_t k = (int64_t)(delta - 1) / hc->w;
        const uint32_t b = (delta - 1) % hc->w;
        int64_t cnt = 0;
        for (int64_t u = hc->word_offsets[k]; u < hc->word_offsets[k + 1]; u++) {
            if ((hc->keys[u] >> b) & 1u) continue;
            const int64_t lo = hc->key_offsets[u], hi = hc->key_offsets[u + 1];
            if (ids) std::memcpy(ids + cnt, hc->ids + lo, sizeof(int32_t) * (size_t)(hi - lo));
            cnt += hi - lo;
        }
        if (ids) std::sort(ids, ids + cnt);  // ascending, like the lattice (reading Q12)
        *count = cnt;
    });
}

// ------------------------------------------------------------------------------ device-level API
skycube_status skycube_ctx_create(int32_t device, skycube_ctx **ctx) {
    if (!ctx) return fail(SKYCUBE_EINVAL, "ctx == NULL");
    *ctx = nullptr;
    return guarded([&] { *ctx = new_ctx(device); });
}

void skycube_ctx_destroy(skycube_ctx *ctx) {
    if (!ctx) return;
    cudaSetDevice(ctx->c.device);
    sky::Ctx &c = ctx->c;
    for (sky::DevBuf *b : {&c.ord, &c.keysum, &c.perm, &c.comp_keys, &c.comp_vals, &c.keys_alt, &c.vals_alt,
                           &c.counts, &c.scan_tmp, &c.flags, &c.scanned, &c.rbuf, &c.minord, &c.nanflag, &c.codes_dm, &c.codes_id,
                           &c.codes_sorted, &c.ord_sorted, &c.ext_id_flag, &c.ext_idx, &c.key_flag, &c.key_idx,
                           &c.ext_ids, &c.p_codes, &c.p_ord, &c.q_codes, &c.q_ord, &c.tie, &c.lat_counts,
                           &c.scan64_tmp, &c.chunks_all, &c.chunks_ext, &c.supers_all, &c.counters, &ctx->input, &ctx->ext8, &ctx->rows32, &ctx->ext_rows32,
                           &ctx->membership, &ctx->offsets, &ctx->ids})
        b->release();
    c.hc.release();
    c.release_sdsc();
    if (ctx->side) cudaStreamDestroy(ctx->side);
    if (ctx->ev_ext) cudaEventDestroy(ctx->ev_ext);
    if (ctx->ev_side) cudaEventDestroy(ctx->ev_side);
    delete ctx;
}

int64_t skycube_ctx_launches(const skycube_ctx *ctx) { return ctx ? ctx->c.L.count : 0; }

skycube_status skycube_ctx_counters(const skycube_ctx *ctx, int64_t *out8) {
    if (!ctx || !out8) return fail(SKYCUBE_EINVAL, "NULL argument");
    return guarded([&] {
        SKY_CUDA(cudaSetDevice(ctx->c.device));
        SKY_CUDA(cudaMemcpy(out8, ctx->c.counters.p, sizeof(int64_t) * 8, cudaMemcpyDeviceToHost));
    });
}

skycube_status skycube_ctx_info(const skycube_ctx *ctx, int64_t *n_ext, uint32_t *words_per_row,
                                uint32_t *exact_mask) {
    if (!ctx) return fail(SKYCUBE_EINVAL, "ctx == NULL");
    if (n_ext) *n_ext = ctx->c.ext_ready ? ctx->c.m : 0;
    if (words_per_row) *words_per_row = ctx->c.W;
    if (exact_mask) *exact_mask = ctx->c.exact_mask;
    return SKYCUBE_OK;
}

skycube_status skycube_dev_prepare(skycube_ctx *ctx, const float *d_points, int64_t n, int32_t d, void *stream) {
    if (!ctx) return fail(SKYCUBE_EINVAL, "ctx == NULL");
    if (d < 1 || d > 16) return fail(SKYCUBE_EINVAL, "d must be in [1, 16]");
    if (n < 1 || n > INT32_MAX) return fail(SKYCUBE_EINVAL, "n must be in [1, INT32_MAX]");
    if (!d_points) return fail(SKYCUBE_EINVAL, "d_points == NULL");
    return guarded([&] {
        SKY_CUDA(cudaSetDevice(ctx->c.device));
        sky::prep_run(ctx->c, d_points, n, d, (cudaStream_t)stream);
    });
}

skycube_status skycube_dev_prepare_dims(skycube_ctx *ctx, const float *d_points, int64_t n, int32_t d, int32_t dim_begin,
                                        int32_t dim_end, uint16_t *d_codes_dm, uint32_t *d_R, uint32_t *d_minord,
                                        void *stream) {
    if (!ctx) return fail(SKYCUBE_EINVAL, "ctx == NULL");
    if (d < 1 || d > 16) return fail(SKYCUBE_EINVAL, "d must be in [1, 16]");
    if (n < 1 || n > INT32_MAX) return fail(SKYCUBE_EINVAL, "n must be in [1, INT32_MAX]");
    if (dim_begin < 0 || dim_end < dim_begin || dim_end > d) return fail(SKYCUBE_EINVAL, "bad dimension slice");
    if (!d_points || (dim_end > dim_begin && (!d_codes_dm || !d_R || !d_minord)))
        return fail(SKYCUBE_EINVAL, "NULL buffer");
    return guarded([&] {
        SKY_CUDA(cudaSetDevice(ctx->c.device));
        sky::prep_dims(ctx->c, d_points, n, d, dim_begin, dim_end, d_codes_dm, d_R, d_minord, (cudaStream_t)stream);
    });
}

skycube_status skycube_dev_prepare_finish(skycube_ctx *ctx, const uint16_t *d_codes_dm, const uint32_t *d_R,
                                          const uint32_t *d_minord, void *stream) {
    if (!ctx) return fail(SKYCUBE_EINVAL, "ctx == NULL");
    if (ctx->c.n < 1 || ctx->c.d < 1) return fail(SKYCUBE_EINVAL, "skycube_dev_prepare_finish before skycube_dev_prepare_dims");
    if (!d_codes_dm || !d_R || !d_minord) return fail(SKYCUBE_EINVAL, "NULL buffer");
    return guarded([&] {
        SKY_CUDA(cudaSetDevice(ctx->c.device));
        sky::prep_finish(ctx->c, d_codes_dm, d_R, d_minord, (cudaStream_t)stream);
    });
}

skycube_status skycube_dev_prefilter(skycube_ctx *ctx, int64_t tile_offset, int64_t tile_step,
                                     uint8_t *d_ext_sorted, void *stream) {
    if (!ctx || !d_ext_sorted) return fail(SKYCUBE_EINVAL, "NULL argument");
    return guarded([&] {
        SKY_CUDA(cudaSetDevice(ctx->c.device));
        sky::prefilter_run(ctx->c, tile_offset, tile_step, d_ext_sorted, (cudaStream_t)stream);
    });
}

skycube_status skycube_dev_set_ext(skycube_ctx *ctx, const uint8_t *d_ext_sorted, int64_t *n_ext, void *stream) {
    if (!ctx || !d_ext_sorted) return fail(SKYCUBE_EINVAL, "NULL argument");
    return guarded([&] {
        SKY_CUDA(cudaSetDevice(ctx->c.device));
        sky::ext_build(ctx->c, d_ext_sorted, (cudaStream_t)stream);
        if (n_ext) *n_ext = ctx->c.m;
    });
}

skycube_status skycube_dev_mdmc(skycube_ctx *ctx, int64_t j_begin, int64_t j_end, uint32_t *d_rows32,
                                uint32_t *d_ext_rows32, void *stream) {
    if (!ctx || !d_rows32) return fail(SKYCUBE_EINVAL, "NULL argument");
    return guarded([&] {
        SKY_CUDA(cudaSetDevice(ctx->c.device));
        sky::mdmc_run(ctx->c, j_begin, j_end, d_rows32, d_ext_rows32, (cudaStream_t)stream);
    });
}

skycube_status skycube_dev_lattice_count(skycube_ctx *ctx, const uint32_t *d_rows32, int64_t j_begin, int64_t j_end,
                                         int64_t *d_totals, void *stream) {
    if (!ctx || !d_rows32 || !d_totals) return fail(SKYCUBE_EINVAL, "NULL argument");
    return guarded([&] {
        sky::Ctx &c = ctx->c;
        if (!c.ext_ready) throw sky::Error{SKYCUBE_EINVAL, "skycube_dev_lattice_count before skycube_dev_set_ext"};
        SKY_CUDA(cudaSetDevice(c.device));
        sky::lattice_count_shard(c, d_rows32, j_begin, j_end, d_totals, (cudaStream_t)stream);
    });
}

skycube_status skycube_dev_lattice_scatter(skycube_ctx *ctx, const uint32_t *d_rows32, int64_t j_begin, int64_t j_end,
                                           const int64_t *d_all_totals, int32_t num_shards, int32_t shard,
                                           int64_t *d_offsets, int32_t *ids, int64_t *total_ids, void *stream) {
    if (!ctx || !d_rows32 || !d_all_totals) return fail(SKYCUBE_EINVAL, "NULL argument");
    if (num_shards < 1 || shard < 0 || shard >= num_shards) return fail(SKYCUBE_EINVAL, "bad shard index");
    return guarded([&] {
        sky::Ctx &c = ctx->c;
        if (!c.ext_ready) throw sky::Error{SKYCUBE_EINVAL, "skycube_dev_lattice_scatter before skycube_dev_set_ext"};
        SKY_CUDA(cudaSetDevice(c.device));
        const int64_t t = sky::lattice_scatter_shard(c, d_rows32, j_begin, j_end, d_all_totals, num_shards, shard,
                                                     d_offsets, ids, (cudaStream_t)stream);
        if (total_ids) *total_ids = t;
    });
}

skycube_status skycube_dev_membership(skycube_ctx *ctx, const uint32_t *d_rows32, int64_t j_begin, int64_t j_end,
                                      int64_t zero_lo, int64_t zero_hi, uint32_t *membership, void *stream) {
    if (!ctx || !d_rows32 || !membership) return fail(SKYCUBE_EINVAL, "NULL argument");
    return guarded([&] {
        sky::Ctx &c = ctx->c;
        if (!c.ext_ready) throw sky::Error{SKYCUBE_EINVAL, "skycube_dev_membership before skycube_dev_set_ext"};
        SKY_CUDA(cudaSetDevice(c.device));
        sky::compact_membership_shard(c, d_rows32, j_begin, j_end, zero_lo, zero_hi, membership, (cudaStream_t)stream);
    });
}

skycube_status skycube_ctx_set_max_level(skycube_ctx *ctx, int32_t max_level) {
    if (!ctx) return fail(SKYCUBE_EINVAL, "ctx == NULL");
    if (max_level < 0 || max_level > 16) return fail(SKYCUBE_EINVAL, "max_level must be in [0, 16]");
    ctx->c.max_level = max_level;
    return SKYCUBE_OK;
}

skycube_status skycube_dev_hashcube(skycube_ctx *ctx, const uint32_t *d_rows32, uint32_t w, int64_t *d_word_offsets,
                                    uint32_t *d_keys, int64_t *d_key_offsets, int32_t *d_ids, int64_t *n_words,
                                    int64_t *total_keys, int64_t *total_ids, void *stream) {
    if (!ctx) return fail(SKYCUBE_EINVAL, "ctx == NULL");
    if (w < 1 || w > 32) return fail(SKYCUBE_EINVAL, "w must be in [1, 32]");
    const bool copy = d_word_offsets || d_keys || d_key_offsets || d_ids;
    if (copy && !(d_word_offsets && d_key_offsets && d_keys && d_ids))
        return fail(SKYCUBE_EINVAL, "all four output buffers are needed");
    if (!copy && !d_rows32) return fail(SKYCUBE_EINVAL, "d_rows32 == NULL");
    return guarded([&] {
        sky::Ctx &c = ctx->c;
        SKY_CUDA(cudaSetDevice(c.device));
        cudaStream_t s = (cudaStream_t)stream;
        sky::HashCubeState &h = c.hc;
        if (!copy) {
            sky::hashcube_build(c, d_rows32, w, s);
        } else {
            if (!h.built || h.w != w) throw sky::Error{SKYCUBE_EINVAL, "no HashCube with this w was built"};
            SKY_CUDA(cudaMemcpyAsync(d_word_offsets, h.woff.p, sizeof(int64_t) * (h.nwords + 1), cudaMemcpyDeviceToDevice, s));
            SKY_CUDA(cudaMemcpyAsync(d_key_offsets, h.koff.p, sizeof(int64_t) * (h.nkeys + 1), cudaMemcpyDeviceToDevice, s));
            if (h.nkeys) SKY_CUDA(cudaMemcpyAsync(d_keys, h.keys32.p, sizeof(uint32_t) * h.nkeys, cudaMemcpyDeviceToDevice, s));
            if (h.nvalid) SKY_CUDA(cudaMemcpyAsync(d_ids, h.vals.p, sizeof(int32_t) * h.nvalid, cudaMemcpyDeviceToDevice, s));
        }
        if (n_words) *n_words = h.nwords;
        if (total_keys) *total_keys = h.nkeys;
        if (total_ids) *total_ids = h.nvalid;
    });
}

skycube_status skycube_dev_compact(skycube_ctx *ctx, const uint32_t *d_rows32, uint32_t *d_membership,
                                   int32_t *d_ext_ids, int64_t *d_offsets, int32_t *d_ids, int64_t *total_ids,
                                   void *stream) {
    if (!ctx || !d_rows32) return fail(SKYCUBE_EINVAL, "NULL argument");
    if (d_ids && !d_offsets) return fail(SKYCUBE_EINVAL, "d_ids needs d_offsets");
    return guarded([&] {
        sky::Ctx &c = ctx->c;
        if (!c.ext_ready) throw sky::Error{SKYCUBE_EINVAL, "skycube_dev_compact before skycube_dev_set_ext"};
        SKY_CUDA(cudaSetDevice(c.device));
        cudaStream_t s = (cudaStream_t)stream;
        if (d_membership) sky::compact_membership(c, d_rows32, d_membership, s);
        if (d_ext_ids && c.m)
            SKY_CUDA(cudaMemcpyAsync(d_ext_ids, c.ext_ids.p, sizeof(int32_t) * c.m, cudaMemcpyDeviceToDevice, s));
        if (d_offsets) {
            int64_t tot = 0;
            if (!d_ids) {
                sky::compact_lattice(c, d_rows32, d_offsets, nullptr, &tot, s);
                if (total_ids) *total_ids = tot;
            } else {
                sky::compact_lattice(c, d_rows32, d_offsets, d_ids, &tot, s);
            }
        }
    });
}

}  // extern "C"
