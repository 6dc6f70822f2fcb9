// common.cuh — shared device/host helpers of the B200 MDMC skycube (sm_100a only).
#pragma once

#include <cuda_runtime.h>
#include <stdint.h>

#include <string>

#if defined(__CUDA_ARCH__) && (__CUDA_ARCH__ < 1000)
#error "this library targets sm_100a (B200) only"
#endif

namespace sky {

constexpr int kMaxD = 16;
constexpr uint32_t kCodeLevels = 32768;  // 15-bit codes (K2); a guard bit per 16-bit SWAR lane
constexpr uint32_t kGuard = 0x80008000u; // guard bits of the two 16-bit lanes of a code word

struct Launches {
    int64_t count = 0;
};

// Error propagation inside the library (converted to skycube_status at the C-ABI).
struct Error {
    int status;  // skycube_status value
    std::string msg;
};

#define SKY_CUDA(call)                                                                          \
    do {                                                                                        \
        cudaError_t _e = (call);                                                                \
        if (_e != cudaSuccess)                                                                  \
            throw ::sky::Error{4, std::string(#call) + ": " + cudaGetErrorString(_e)};          \
    } while (0)

#define SKY_LAUNCH_CHECK()                                                                      \
    do {                                                                                        \
        cudaError_t _e = cudaGetLastError();                                                    \
        if (_e != cudaSuccess)                                                                  \
            throw ::sky::Error{4, std::string("kernel launch: ") + cudaGetErrorString(_e)};     \
    } while (0)

// Process-wide tuning / test overrides (skycube_set_tuning in the C-ABI; never read from the environment in
// the launch path).  0 = automatic.
struct Tuning {
    int k3_design = 0;      // 'A' or 'O': force a K3 design
    int k3_tpc = 0;         // force K3 tasks per CTA (design A)
    int k3_warps = 0;       // K3 design A consumer warps: 0 = automatic (24 at d = 12, else 16), or 16 / 24
    int k3_mode = -1;       // force a K3 state mode (0, 1, 2); -1 = automatic
    int share_devices = 0;  // 1: multi-GPU ranks may share devices (tests of the k-rank logic on one GPU)
};
Tuning &tuning();

inline uint32_t words_per_row(int d) { return d >= 5 ? (1u << (d - 5)) : 1u; }
inline int dpad_of(int d) { return ((d + 3) / 4) * 4; }  // codes padded to groups of 4 dims
inline int64_t ceil_div(int64_t a, int64_t b) { return (a + b - 1) / b; }
__device__ __forceinline__ int64_t ceil_div_dev(int64_t a, int64_t b) { return (a + b - 1) / b; }

// ------------------------------------------------------------------------------ sort / scan API
// Stable LSD radix sort of (key, value) pairs on the low `bits` bits of the 64-bit keys.
// Buffers: keys/vals in, sorted back into keys/vals (ping-pong through tmp buffers).
struct SortScratch {
    void *keys_alt = nullptr;
    void *vals_alt = nullptr;
    void *counts = nullptr;     // [256 * nblocks] uint32
    void *scan_tmp = nullptr;   // scan scratch
    size_t keys_alt_bytes = 0, vals_alt_bytes = 0, counts_bytes = 0, scan_tmp_bytes = 0;
};

size_t radix_scratch_counts(int64_t n);
void radix_sort_u64(uint64_t *keys, uint32_t *vals, int64_t n, int bits, uint64_t *keys_alt,
                    uint32_t *vals_alt, uint32_t *counts, void *scan_tmp, cudaStream_t st,
                    Launches &L);

// Exclusive scan of n uint32 (out may alias in).  Returns nothing; total via out[n-1]+in[n-1] or
// by the caller.  tmp must hold scan_tmp_bytes(n) bytes.
size_t scan_tmp_bytes(int64_t n);
void exclusive_scan_u32(const uint32_t *in, uint32_t *out, int64_t n, void *tmp, cudaStream_t st,
                        Launches &L);
void exclusive_scan_u64(const uint64_t *in, uint64_t *out, int64_t n, void *tmp, cudaStream_t st,
                        Launches &L);

}  // namespace sky
