// tile_stream.cuh — TMA bulk-copy (cp.async.bulk) + mbarrier double buffering of competitor tiles.
//
// Every K1/K3 CTA streams the same competitor array from L2 (it is read by all CTAs and stays
// L2-resident: <= 64 MB of codes).  One elected thread issues a 1-D bulk copy of tile t+2 into the
// stage that tile t just released; consumers wait on the stage's mbarrier (phase parity).
#pragma once

#include <stdint.h>

namespace sky {

__device__ __forceinline__ uint32_t smem_u32(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }

__device__ __forceinline__ void mbar_init(uint64_t *bar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}

__device__ __forceinline__ void mbar_fence_init() {
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}

__device__ __forceinline__ void mbar_arrive_expect_tx(uint64_t *bar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes) : "memory");
}

__device__ __forceinline__ void bulk_g2s(void *dst, const void *src, uint32_t bytes, uint64_t *bar) {
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                     smem_u32(dst)),
                 "l"(src), "r"(bytes), "r"(smem_u32(bar))
                 : "memory");
}

__device__ __forceinline__ void mbar_wait(uint64_t *bar, uint32_t parity) {
    const uint32_t addr = smem_u32(bar);
    uint32_t done;
    do {
        asm volatile(
            "{\n .reg .pred p;\n mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n selp.u32 %0, 1, 0, p;\n}\n"
            : "=r"(done)
            : "r"(addr), "r"(parity)
            : "memory");
    } while (!done);
}

// Producer-side wait (the stage the producer refills is S tiles behind the consumers, so its wake-up latency
// is hidden): try_wait with a suspend-time hint, the hardware deschedules the waiting producer warp instead of
// letting it poll.  It replaces a nanosleep back-off whose polling loop was ~5% of K3's issued instructions at
// H (ncu source view); measured: K1 13.1 -> 12.8 ms at H, K3 unchanged.  (Precomputed 32-bit barrier
// addresses, and the same hint on the consumers' waits, each measured ~2% slower in K3 and were reverted.)
__device__ __forceinline__ void mbar_wait_sleep(uint64_t *bar, uint32_t parity) {
    const uint32_t addr = smem_u32(bar);
    uint32_t done;
    do {
        asm volatile(
            "{\n .reg .pred p;\n mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2, %3;\n selp.u32 %0, 1, 0, p;\n}\n"
            : "=r"(done)
            : "r"(addr), "r"(parity), "r"(200000u)
            : "memory");
    } while (!done);
}

// 32-bit shared-window forms for kernels that keep barrier addresses in registers (design O of K3).
__device__ __forceinline__ void mbar_wait_s(uint32_t addr, uint32_t parity) {
    uint32_t done;
    do {
        asm volatile(
            "{\n .reg .pred p;\n mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n selp.u32 %0, 1, 0, p;\n}\n"
            : "=r"(done)
            : "r"(addr), "r"(parity)
            : "memory");
    } while (!done);
}
__device__ __forceinline__ void mbar_arrive_s(uint32_t addr) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(addr) : "memory");
}

// Double-buffered stream of fixed-size tiles (bytes multiple of 16, 16-B aligned source).
struct TileStream2 {
    uint64_t *bar;  // [2] in shared memory
    uint32_t *buf;  // [2][tile_words] in shared memory
    uint32_t tile_words;

    __device__ __forceinline__ uint32_t *stage(int64_t t) const { return buf + (t & 1) * tile_words; }

    // thread 0 only
    __device__ __forceinline__ void init() const {
        mbar_init(&bar[0], 1);
        mbar_init(&bar[1], 1);
        mbar_fence_init();
    }
    // thread 0 only
    __device__ __forceinline__ void issue(const uint32_t *src_tiles, int64_t t) const {
        const uint32_t bytes = tile_words * 4u;
        mbar_arrive_expect_tx(&bar[t & 1], bytes);
        bulk_g2s(stage(t), src_tiles + t * (int64_t)tile_words, bytes, &bar[t & 1]);
    }
    __device__ __forceinline__ void wait(int64_t t) const { mbar_wait(&bar[t & 1], (uint32_t)((t >> 1) & 1)); }
};

__device__ __forceinline__ void mbar_arrive(uint64_t *bar) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}

// S-stage ring of fixed-size tiles with full (TMA complete_tx) and empty (consumer arrival) barriers.
// Consumers: wait(t), read stage(t), then one arrival per consumer unit on release(t).
// Producer (one thread): before issuing tile t >= S, waits until tile t-S released its stage.
template <int S>
struct TileRing {
    uint64_t *full;   // [S]
    uint64_t *empty;  // [S]
    uint32_t *buf;    // [S][tile_words]
    uint32_t tile_words;

    __device__ __forceinline__ uint32_t *stage(int64_t t) const { return buf + (uint32_t)(t % S) * tile_words; }
    __device__ __forceinline__ void init(uint32_t consumers) const {
        for (int i = 0; i < S; i++) {
            mbar_init(&full[i], 1);
            mbar_init(&empty[i], consumers);
        }
        mbar_fence_init();
    }
    __device__ __forceinline__ void issue(const uint32_t *src_tiles, int64_t t) const {
        const int s = (int)(t % S);
        if (t >= S) mbar_wait_sleep(&empty[s], (uint32_t)(((t / S) - 1) & 1));
        const uint32_t bytes = tile_words * 4u;
        mbar_arrive_expect_tx(&full[s], bytes);
        bulk_g2s(buf + (uint32_t)s * tile_words, src_tiles + t * (int64_t)tile_words, bytes, &full[s]);
    }
    // Two-segment tile: words [0, na) from a + t*na, then words [na, na+nb) from b + t*nb (tile_words = na+nb).
    __device__ __forceinline__ void issue2(const uint32_t *a, uint32_t na, const uint32_t *b, uint32_t nb,
                                           int64_t t) const {
        const int s = (int)(t % S);
        if (t >= S) mbar_wait_sleep(&empty[s], (uint32_t)(((t / S) - 1) & 1));
        mbar_arrive_expect_tx(&full[s], (na + nb) * 4u);
        uint32_t *dst = buf + (uint32_t)s * tile_words;
        bulk_g2s(dst, a + t * (int64_t)na, na * 4u, &full[s]);
        bulk_g2s(dst + na, b + t * (int64_t)nb, nb * 4u, &full[s]);
    }
    __device__ __forceinline__ void wait(int64_t t) const { mbar_wait(&full[t % S], (uint32_t)((t / S) & 1)); }
    __device__ __forceinline__ void release(int64_t t) const { mbar_arrive(&empty[t % S]); }

    // Filtered streams: the producer fills ring slot k (the k-th streamed tile) with source tile t.
    __device__ __forceinline__ void wait_empty(int64_t slot) const {
        if (slot >= S) mbar_wait_sleep(&empty[slot % S], (uint32_t)(((slot / S) - 1) & 1));
    }
    __device__ __forceinline__ void issue2_slot(const uint32_t *a, uint32_t na, const uint32_t *b, uint32_t nb, int64_t t,
                                                int64_t slot) const {
        const int s = (int)(slot % S);
        mbar_arrive_expect_tx(&full[s], (na + nb) * 4u);
        uint32_t *dst = buf + (uint32_t)s * tile_words;
        bulk_g2s(dst, a + t * (int64_t)na, na * 4u, &full[s]);
        bulk_g2s(dst + na, b + t * (int64_t)nb, nb * 4u, &full[s]);
    }
    // completes the slot's phase without data (an end-of-stream marker stored in shared memory before it)
    __device__ __forceinline__ void arrive_full(int64_t slot) const { mbar_arrive(&full[slot % S]); }
};

// Named barrier 1 over the consumer warps (the producer warp has left the CTA-wide barrier 0).
__device__ __forceinline__ void consumer_sync(int nthreads) {
    asm volatile("bar.sync 1, %0;" ::"r"(nthreads) : "memory");
}

}  // namespace sky
