// ctx.cuh — per-device context: grow-only device workspace and the phase launchers.
#pragma once

#include "common.cuh"

namespace sky {

struct DevBuf {
    void *p = nullptr;
    size_t bytes = 0;
    template <typename T>
    T *as() const { return reinterpret_cast<T *>(p); }
    void ensure(size_t b) {
        if (b <= bytes) return;
        if (p) cudaFree(p);
        p = nullptr;
        bytes = 0;
        size_t want = b + b / 8 + 256;
        cudaError_t e = cudaMalloc(&p, want);
        if (e != cudaSuccess) {
            cudaGetLastError();
            p = nullptr;
            throw Error{3, std::string("cudaMalloc(") + std::to_string(want) + "): " + cudaGetErrorString(e)};
        }
        bytes = want;
    }
    void release() {
        if (p) cudaFree(p);
        p = nullptr;
        bytes = 0;
    }
};

// HashCube of the last skycube_dev_hashcube / skycube_build_hashcube call (K5, k5_hashcube.cu)
struct HashCubeState {
    bool built = false;
    uint32_t w = 0;
    int64_t nwords = 0, nvalid = 0, nkeys = 0;
    DevBuf keys, vals, keys_alt, vals_alt, counts, scan_tmp, nvalid_dev;  // items (word, key) -> id, sorted
    DevBuf ukeys;   // u64 [nkeys]   distinct composites (k << w) | key
    DevBuf keys32;  // u32 [nkeys]   keys
    DevBuf koff;    // i64 [nkeys+1] first item of each key (ids = vals[koff[u] .. koff[u+1]))
    DevBuf woff;    // i64 [nwords+1] first key of each word
    void release() {
        for (DevBuf *b : {&keys, &vals, &keys_alt, &vals_alt, &counts, &scan_tmp, &nvalid_dev, &ukeys, &keys32, &koff, &woff})
            b->release();
        built = false;
    }
};

struct Ctx {
    int device = 0;
    int num_sms = 148;
    Launches L;
    // problem
    int64_t n = 0;
    int d = 0, dp = 0;
    uint32_t W = 1;
    uint32_t exact_mask = 0;    // bit i <=> the codes of dimension i are injective (dense ranks)
    uint32_t R[kMaxD] = {0};    // distinct values per dimension
    uint64_t cshift = 0;        // coarse-code shift of dimension i in bits 4i..4i+3 (K3 corner tests)
    int64_t m = 0;              // |S+(P)|
    int max_level = 0;          // partial skycube (Appendix A.2): report only |delta| <= max_level (0 = d)
    bool prepared = false, ext_ready = false;
    // preparation (all n points)
    DevBuf ord;         // u32 [n*d]   order-preserving keys, id order
    DevBuf keysum;      // u64 [n]     sum of keys (Λ2), later sorted
    DevBuf perm;        // u32 [n]     sorted position -> id
    DevBuf comp_keys;   // u64 [n*d]   (dim << 32) | key, sorted per dimension
    DevBuf comp_vals;   // u32 [n*d]   point id
    DevBuf keys_alt, vals_alt, counts, scan_tmp;
    DevBuf flags;       // u32 [n*d]
    DevBuf scanned;     // u32 [n*d]
    DevBuf rbuf;        // u32 [kMaxD]
    DevBuf minord;      // u32 [kMaxD]  key of each dimension's minimum value
    DevBuf nanflag;     // u32 [1]
    DevBuf codes_dm;    // u16 [d][n]  codes, dim-major (prep_dims output on one GPU)
    DevBuf codes_id;    // u16 [n*dp]  id order
    DevBuf codes_sorted;// u16 [npad*dp]  static-tree (Morton) order, padded to whole chunk tiles
    DevBuf ord_sorted;  // u32 [n*d]      static-tree order
    // S+ (m points)
    DevBuf ext_id_flag, ext_idx, key_flag, key_idx;  // u32 [n]
    DevBuf ext_ids;     // i32 [m] ascending
    DevBuf p_codes;     // u16 [m*dp]  S+ in id order (MDMC tasks)
    DevBuf p_ord;       // u32 [m*d]
    DevBuf q_codes;     // u16 [mpad*dp]  S+ in static-tree order (MDMC competitor stream)
    DevBuf q_ord;       // u32 [m*d]
    DevBuf tie;         // u32 tiled rows: tie contributions to B_{p notin S}
    DevBuf chunks_all;  // u32 [n/32][kRecAll][cw]  chunk records of all points (K1 competitors)
    DevBuf chunks_ext;  // u32 [m/32][rec_ext_words(cw)]  chunk records of S+ with coarse corners (K3 competitors)
    DevBuf chunk_keys, chunk_perm, q_codes_alt, q_ord_alt;  // chunk visiting order (strongest corner first)
    DevBuf supers_all;  // u32 [tiles][super_words(cw)]  lower corner of each tile of 16 chunks (K1)
    int64_t nchunks_all = 0, nchunks_ext = 0;
    DevBuf lat_counts;  // u64 [2^d * nchunks]
    DevBuf counters;    // u64 [8]: K1 box tests, K1 pair tests, K3 box tests, K3 pair tests, K3 misses
    DevBuf scan64_tmp;
    HashCubeState hc;
    // SDSC comparator (sdsc.cu)
    DevBuf sdsc_prev, sdsc_next, sdsc_ids_tmp, sdsc_tab, sdsc_items, sdsc_keys, sdsc_vals, sdsc_keys_alt, sdsc_vals_alt,
        sdsc_counts, sdsc_scan, sdsc_status, sdsc_flags, sdsc_cnt, sdsc_lat, sdsc_ids;
    void release_sdsc() {
        for (DevBuf *b : {&sdsc_prev, &sdsc_next, &sdsc_ids_tmp, &sdsc_tab, &sdsc_items, &sdsc_keys, &sdsc_vals,
                          &sdsc_keys_alt, &sdsc_vals_alt, &sdsc_counts, &sdsc_scan, &sdsc_status, &sdsc_flags,
                          &sdsc_cnt, &sdsc_lat, &sdsc_ids})
            b->release();
    }
};

// prep.cu
void prep_run(Ctx &c, const float *d_points, int64_t n, int d, cudaStream_t st);
// the two halves of prep_run (multi-GPU prepare: every rank the codes of a slice of the dimensions, then an
// all-gather of the codes, then prep_finish on every rank)
void prep_dims(Ctx &c, const float *d_points, int64_t n, int d, int db, int de, uint16_t *codes_dm, uint32_t *R,
               uint32_t *minord, cudaStream_t st);
void prep_finish(Ctx &c, const uint16_t *codes_dm, const uint32_t *R, const uint32_t *minord, cudaStream_t st);
void ext_build(Ctx &c, const uint8_t *d_ext_sorted, cudaStream_t st);
void or_flags(Ctx &c, const uint8_t *stage, int k, int64_t n, uint8_t *out, cudaStream_t st);
// k1_prefilter.cu
void prefilter_run(Ctx &c, int64_t tile_offset, int64_t tile_step, uint8_t *d_ext_sorted, cudaStream_t st);
// k3_mdmc.cu
// host_membership (nullable): pinned host array [n][W] that also receives every S+ row by point id (zero-copy)
void mdmc_run(Ctx &c, int64_t j_begin, int64_t j_end, uint32_t *d_rows32, uint32_t *d_ext_rows32, cudaStream_t st,
              uint32_t *host_membership = nullptr);
// k4_compact.cu
void compact_membership(Ctx &c, const uint32_t *rows32, uint32_t *membership, cudaStream_t st);
// zero rows of the points outside S+ in a (host-mapped) membership array [n][W] (zero-copy path)
void membership_zero_outside(Ctx &c, uint32_t *membership, cudaStream_t st);
void compact_lattice(Ctx &c, const uint32_t *rows32, int64_t *offsets, int32_t *ids, int64_t *total_ids,
                     cudaStream_t st);
// multi-GPU shards of K4 (S+ tasks [j0, j1), j0 a multiple of 32): count -> exchange totals -> scatter
void lattice_count_shard(Ctx &c, const uint32_t *rows32, int64_t j0, int64_t j1, int64_t *d_totals, cudaStream_t st);
int64_t lattice_scatter_shard(Ctx &c, const uint32_t *rows32, int64_t j0, int64_t j1, const int64_t *all_totals, int k,
                              int rank, int64_t *offsets, int32_t *ids, cudaStream_t st);
void compact_membership_shard(Ctx &c, const uint32_t *rows32, int64_t j0, int64_t j1, int64_t zlo, int64_t zhi,
                              uint32_t *membership, cudaStream_t st);
// sdsc.cu: Alg. 2 over the installed S+; lattice into d_offsets / *d_ids (context-owned), rows into
// d_membership (nullable); returns the number of ids
int64_t sdsc_run(Ctx &c, int64_t *d_offsets, uint32_t *d_membership, cudaStream_t st, int32_t **d_ids);
// k5_hashcube.cu
int64_t hashcube_words(int d, uint32_t w);
void hashcube_build(Ctx &c, const uint32_t *rows32, uint32_t w, cudaStream_t st);

constexpr int64_t kQPad = 21504;     // competitor stream padded to whole MDMC tiles (16, 24, 28 or 32 chunks)
constexpr int64_t kChunkTilePad = 512;  // extra never-better points so chunk tiles (16 chunks) are whole
constexpr int kTileChunks = 16;         // chunks per competitor tile (one super-chunk of 512 points)
constexpr int kSubSize = 4;             // points per sub-chunk (K3 level below the chunk)
constexpr int kRecAll = 33;             // K1 chunk record rows: 32 points + corner
// K3 chunk records: the 32 members' 15-bit code words (cw words each, the pair pass), then the chunk's lower
// corner and the lower corners of its 8 sub-chunks as COARSE codes: 7 bits per dimension, four dimensions per
// 32-bit word (kCoarseWords words per row, d <= 16), for the corner tests (box and sub-chunk passes).  The
// coarse code of dimension i is min(code >> cshift_i, 127), cshift_i the smallest shift that maps the
// dimension's codes into 7 bits (0 when it has <= 128 distinct values): monotone, so a coarse lower corner
// below p in dimension i is implied by the fine one and every corner test stays sound (Λ3, Λ4).
constexpr int kCoarseWords = 4;
constexpr int kCoarseRows = 1 + 32 / kSubSize;  // chunk corner + 8 sub-chunk corners
__host__ __device__ inline int rec_ext_words(int cw) { return 32 * cw + kCoarseRows * kCoarseWords; }
inline int super_words(int cw) { return (cw + 3) & ~3; }  // super-corner record words (16-byte multiple)

}  // namespace sky
