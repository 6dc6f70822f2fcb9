/*
 * skycube.h — C-ABI of the B200-native point-based MDMC skycube (Bøgh, Chester, Šidlauskas, Assent,
 * "Template Skycube Algorithms for Heterogeneous Parallelism on Multicore and GPU Architectures",
 * SIGMOD'17).  Citations "Lnnn" are lines of the paper transcript.
 *
 * What is computed (Def. 1-3):
 *   Input P: n points over d dimensions, float32, smaller is better (footnote 2, L114).
 *   For every subspace 0 < delta < 2^d (bit i of delta <=> dimension i, L76), the subspace skyline
 *     S_delta(P) = { p : no q in P dominates p in delta }, where q dominates p in delta iff
 *     (B_{q=p} & delta) != delta and (B_{q<=p} & delta) == delta (Def. 1).
 *   The skycube (Def. 3) is returned in two forms:
 *     - per point, its membership bitmap (the paper's B_{p in S}, L84, here UNSHIFTED: bit delta, not
 *       bit delta-1);
 *     - per subspace, the ascending id list of S_delta(P) (the lattice of Fig. 1a).
 *   Method: Alg. 3 (MDMC, L318-324) on the GPU: S+(P) prefilter (line 2), then one data-parallel task
 *   per p in S+(P) computing B_{p notin S} and B_{p notin S+} (lines 3-12), then compaction.
 *
 * Value semantics (readings Q9-Q12): IEEE binary32 compares only; -0 == +0; +-inf are
 * ordinary values; NaN is rejected (SKYCUBE_ENAN); equal points never dominate each other; ids are
 * the row indices of `points` (footnote 1, L78).
 *
 * Errors: every entry point returns a skycube_status; on any error the output struct is zeroed and
 * owns nothing; skycube_last_error() gives a thread-local detail string.  All calls are serialised
 * by a process-wide mutex.
 */
#ifndef SKYCUBE_H
#define SKYCUBE_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
    SKYCUBE_OK = 0,
    SKYCUBE_EINVAL = 1, /* bad argument: NULL pointer with n > 0, d outside [1,16], n > INT32_MAX */
    SKYCUBE_ENAN = 2,   /* a NaN in the input */
    SKYCUBE_ENOMEM = 3, /* host or device allocation failed */
    SKYCUBE_ECUDA = 4,  /* CUDA runtime / kernel error */
    SKYCUBE_ENCCL = 5,  /* reserved for a collective-library error; not returned today: the
                           single-process num_gpus path exchanges with CUDA peer copies (errors: ECUDA) and
                           the per-rank path leaves collectives to the caller (torch.distributed / NCCL) */
    SKYCUBE_ENODEV = 6  /* no sm_100 device visible */
} skycube_status;

/* flags for skycube_opts.flags */
#define SKYCUBE_NO_LISTS 0x1u          /* skip the per-subspace id lists (rows only) */
#define SKYCUBE_EXT_MEMBERSHIP 0x2u    /* debug: also return B_{p in S+} rows (ext_membership) */

typedef struct {
    int32_t d;                 /* 1..16 */
    int64_t n;                 /* number of points */
    int64_t n_ext;             /* |S+(P)|: full-space extended skyline size (Def. 2, delta = 2^d-1) */
    int32_t *ext_ids;          /* [n_ext] ascending ids of S+(P) */
    uint32_t words_per_row;    /* W = max(1, 2^d / 32) */
    uint32_t *membership;      /* [n * W] row p, bit delta (word delta>>5, bit delta&31) <=> p in S_delta(P);
                                  bit 0 always 0; rows of points outside S+(P) are all zero (L106) */
    uint32_t *ext_membership;  /* [n * W] or NULL: bit delta <=> p in S+_delta(P) (SKYCUBE_EXT_MEMBERSHIP) */
    int64_t *cuboid_offsets;   /* [2^d + 1] or NULL (NO_LISTS): ids of S_delta are
                                  cuboid_ids[off[delta] .. off[delta+1]); off[0] = off[1] = 0 */
    int32_t *cuboid_ids;       /* [off[2^d]] ascending within each delta */
} skycube_result;

typedef struct {
    int32_t num_gpus;     /* 0 or 1 = one GPU; k > 1 = single-process sharding over devices device .. device+k-1:
                             prepare replicated, K1 blocks and K3 task groups split k ways, S+ flags and rows
                             gathered on `device` by peer copies (NVLink); same output bytes as one GPU.
                             ENODEV if fewer devices are visible; not with SKYCUBE_EXT_MEMBERSHIP (EINVAL) */
    int32_t device;       /* CUDA device ordinal to use (the first one when num_gpus > 1) */
    uint32_t flags;       /* SKYCUBE_* flags */
    int32_t max_level;    /* partial skycube (Appendix A.2): 0 = full skycube; d' in [1, d] =
                             only the subspaces with |delta| <= d' are computed and reported -- membership
                             bits of every delta with |delta| > d' are 0 and their lists are empty
                             (reading P1: "no correctness guarantee is offered for the skyline
                             of said delta", L1248) */
} skycube_opts;

typedef struct {
    double ms_total;       /* whole call, host clock */
    double ms_h2d, ms_validate, ms_sort, ms_codes, ms_prefilter, ms_mdmc, ms_compact, ms_d2h; /* CUDA events */
    int64_t n_ext;         /* |S+(P)| */
    int64_t pairs;         /* n_ext * (n_ext - 1): ordered S+ pairs tested by MDMC */
    int64_t total_ids;     /* sum over delta of |S_delta(P)| */
    int32_t kernel_launches;
    double ms_comm;        /* multi-GPU exchange (flag and row gathers), host clock; 0 on one GPU */
    int64_t exact_dts;     /* pairs that reached the exact dominance test of Alg. 3 line 10 (K3 misses) */
    int64_t expansions;    /* contributing competitors expanded into the state (Alg. 3 lines 11-12) */
    int32_t num_gpus;      /* devices the build ran on */
} skycube_stats;

/* Build the skycube of the host array points[n*d] (row-major, row = id, column i = dimension i).
 * `points` is caller-owned and only read.  `out` is caller-provided; every buffer in it is allocated
 * by the library (pinned host memory) and must be released with skycube_free.  n == 0 returns OK
 * with empty outputs.  Uses CUDA device 0. */
skycube_status skycube_build(const float *points, int64_t n, int32_t d, skycube_result *out);

/* As skycube_build with options (NULL = defaults) and optional per-phase statistics (NULL = none). */
skycube_status skycube_build_ex(const float *points, int64_t n, int32_t d, const skycube_opts *opts,
                                skycube_result *out, skycube_stats *stats);

/* Release every buffer of `out` and zero it.  Idempotent; safe on a zeroed struct. */
void skycube_free(skycube_result *out);

/* SDSC comparator (Alg. 2, §4.2.2): the paper's lattice-based template -- a
 * top-down traversal where every cuboid delta is computed as a parallel skyline over its cheapest parent's
 * extended skyline L[parent] U L+[parent] (reading S1: parent = the immediate superset with the fewest
 * points, ties to the smaller delta').  Same inputs, outputs, conventions and errors as skycube_build_ex
 * (membership rows, ext_ids and the lattice; opts: device only).  Not the product path: it exists to
 * compare MDMC with the paper's alternative on the same GPU, and its cost grows with 2^d cuboid passes. */
skycube_status skycube_build_sdsc(const float *points, int64_t n, int32_t d, const skycube_opts *opts,
                                  skycube_result *out, skycube_stats *stats);

/* ------------------------------------------------------------------------------------------------
 * HashCube output (Alg. 3 lines 1 and 13, L320; Appendix B.1; Fig. 1b).
 * Point p is represented by B_{p notin S}: 2^d - 1 bits, bit delta-1 set <=> p is dominated in delta
 * (the shifted order of L84).  It is cut into n_words = ceil((2^d - 1) / w) words of w bits (word k =
 * subspaces k*w+1 .. k*w+w; the last word may be shorter) and word k is hashed by h_k: key = the word's
 * value, value = the ids of the points with that key.  A point whose word is all set (dominated in all
 * of the word's subspaces) is not stored (L1278); points outside S+(P) are never stored.
 * The hash maps are returned as sorted arrays (reading H1): the keys of word k are
 * keys[word_offsets[k] .. word_offsets[k+1]) ascending, the ids of key u are
 * ids[key_offsets[u] .. key_offsets[u+1]) ascending.
 * Retrieval of S_delta (L1280, reading Q6): the lists of h_{(delta-1)/w} whose key has bit (delta-1) % w
 * NOT set -- see skycube_hashcube_query.
 * ------------------------------------------------------------------------------------------------ */
typedef struct {
    int32_t d;
    uint32_t w;               /* word length, 1..32 (the paper's GPU HashCube uses 32, L158) */
    int64_t n;                /* number of points */
    int64_t n_ext;            /* |S+(P)| */
    int64_t n_words;          /* ceil((2^d - 1) / w) hash functions */
    int64_t total_keys;       /* distinct (word, key) pairs stored */
    int64_t total_ids;        /* stored ids: at most n_ext * n_words */
    int64_t *word_offsets;    /* [n_words + 1] */
    uint32_t *keys;           /* [total_keys]  bit b <=> dominated in subspace k*w + b + 1 */
    int64_t *key_offsets;     /* [total_keys + 1] */
    int32_t *ids;             /* [total_ids] */
} skycube_hashcube;

/* Build the skycube of points[n*d] (as skycube_build) and return it as a HashCube with word length w.
 * opts (nullable): device, max_level (partial skycube: subspaces above d' are reported as dominated,
 * which the HashCube then compresses away); flags and num_gpus are ignored.  Buffers are pinned host
 * memory owned by the library; release with skycube_hashcube_free.  Errors as skycube_build_ex, plus
 * EINVAL for w outside [1, 32] and ENOMEM when n_ext * n_words >= 2^32. */
skycube_status skycube_build_hashcube(const float *points, int64_t n, int32_t d, uint32_t w, const skycube_opts *opts,
                                      skycube_hashcube *out, skycube_stats *stats);

/* Release every buffer of `hc` and zero it.  Idempotent; safe on a zeroed struct. */
void skycube_hashcube_free(skycube_hashcube *hc);

/* Subspace skyline query on a HashCube (the read path, L1280): *count = |S_delta(P)|; if ids != NULL it
 * must hold *count entries (call once with ids == NULL to size it) and receives the ids ascending.
 * Host-side; EINVAL for delta outside [1, 2^d - 1] or a zeroed hc. */
skycube_status skycube_hashcube_query(const skycube_hashcube *hc, uint32_t delta, int32_t *ids, int64_t *count);

const char *skycube_strerror(skycube_status s);
const char *skycube_last_error(void);   /* thread-local detail of the last error */

/* Process-wide tuning / test overrides (performance only: every setting gives the same output bytes).
 * Keys: "k3_design" ('A', 'O' or 0 = automatic), "k3_tpc" (K3 tasks per CTA, 0 = automatic), "k3_mode"
 * (K3 state mode 0/1/2, -1 = automatic), "k3_warps" (K3 design A consumer warps: 0 = automatic (24 at d = 12, else 16), 16 forces 16),
 * "share_devices" (1: num_gpus ranks may share devices, so the
 * multi-GPU logic can be tested on one GPU), "reset" (all automatic).  EINVAL for an unknown key or value.
 * Serialised with the build calls. */
skycube_status skycube_set_tuning(const char *key, int32_t value);

/* ------------------------------------------------------------------------------------------------
 * Device-resident entry points (used by the per-rank multi-GPU driver and the benchmark).
 * All pointers here are DEVICE pointers on the context's device; `stream` is a cudaStream_t passed as
 * void* (NULL = legacy default stream).  A context owns a grow-only device workspace reused across
 * calls; it is not thread-safe (one context per thread / rank).
 * ------------------------------------------------------------------------------------------------ */
typedef struct skycube_ctx skycube_ctx;

skycube_status skycube_ctx_create(int32_t device, skycube_ctx **ctx);
void skycube_ctx_destroy(skycube_ctx *ctx);

/* Phase 1 (replicated on every rank): validate (K0: NaN -> ENAN, -0 -> +0, order-preserving keys),
 * compute per-dimension 15-bit monotone codes (K2), and put the points in static-tree order (Morton order
 * of the codes: the leaf order of the paper's global-pivot tree, L338) with 32-point chunk records.
 * d_points: [n*d] float32 row-major on the device. */
skycube_status skycube_dev_prepare(skycube_ctx *ctx, const float *d_points, int64_t n, int32_t d, void *stream);

/* The two halves of skycube_dev_prepare, for a preparation sharded over the ranks of a multi-GPU run (SURVEY
 * §8(e); the per-dimension ranks of K2 are independent across dimensions, so rank r computes the codes of its
 * slice of the dimensions and the ranks all-gather them):
 *
 * skycube_dev_prepare_dims: K0 (validation, order-preserving keys of EVERY dimension, kept in the context) and
 *   K2 on the dimensions [dim_begin, dim_end) only: d_codes_dm (device, uint16 [dim_end - dim_begin][n],
 *   dim-major, caller-owned) receives their 15-bit codes; d_R / d_minord (device, uint32 [d], caller-owned)
 *   receive, at the indices dim_begin .. dim_end - 1, the number of distinct values and the minimum order key
 *   of each dimension.  dim_begin == dim_end runs K0 only.  Errors as skycube_dev_prepare (ENAN on NaN).
 * skycube_dev_prepare_finish: completes the preparation from every dimension's codes: d_codes_dm uint16
 *   [d][n] (dim-major), d_R and d_minord uint32 [d], all device and caller-owned (read only).  Afterwards the
 *   context is in the state skycube_dev_prepare leaves it in.  EINVAL before skycube_dev_prepare_dims. */
skycube_status skycube_dev_prepare_dims(skycube_ctx *ctx, const float *d_points, int64_t n, int32_t d, int32_t dim_begin,
                                        int32_t dim_end, uint16_t *d_codes_dm, uint32_t *d_R, uint32_t *d_minord,
                                        void *stream);
skycube_status skycube_dev_prepare_finish(skycube_ctx *ctx, const uint16_t *d_codes_dm, const uint32_t *d_R,
                                          const uint32_t *d_minord, void *stream);

/* Phase 2: extended-skyline prefilter (K1).  The prepared (static-tree) positions are cut into blocks of
 * 512 (one K1 CTA each); this call processes the blocks b with b % tile_step == tile_offset (interleaving balances ranks).
 * Writes d_ext_sorted[s] = 1 iff the point at prepared position s is in S+(P), 0 otherwise, for the
 * positions of those blocks only.  d_ext_sorted: [n] uint8 device buffer owned by the caller. */
skycube_status skycube_dev_prefilter(skycube_ctx *ctx, int64_t tile_offset, int64_t tile_step,
                                     uint8_t *d_ext_sorted, void *stream);

/* Phase 3: install the S+ flags (d_ext_sorted: [n] complete, identical on every rank) and build the
 * S+ structures; returns n_ext. */
skycube_status skycube_dev_set_ext(skycube_ctx *ctx, const uint8_t *d_ext_sorted, int64_t *n_ext, void *stream);

/* Phase 4: MDMC (K3) for the S+ points j in [j_begin, j_end) (id-ascending S+ index; j_begin a
 * multiple of 32, j_end <= n_ext).  Writes their membership rows into d_rows32, the tiled layout
 * d_rows32[(j/32)*W*32 + w*32 + j%32] = word w of the membership bitmap of S+ point j
 * (buffer size ceil(n_ext/32)*32*W uint32).  d_ext_rows32 (same layout, may be NULL) receives the
 * extended-skyline rows B_{p in S+} (debug / tests). */
skycube_status skycube_dev_mdmc(skycube_ctx *ctx, int64_t j_begin, int64_t j_end, uint32_t *d_rows32,
                                uint32_t *d_ext_rows32, void *stream);

/* Phase 5: compaction (K4): from the complete tiled rows of all S+ points, write
 * d_membership[n*W] (NULL = skip), d_ext_ids[n_ext] (NULL = skip), and, unless d_offsets == NULL,
 * the lattice: d_offsets[2^d+1] and d_ids[total_ids].  Call first with d_ids == NULL to obtain
 * *total_ids (offsets are written), then with d_ids of that size. */
skycube_status skycube_dev_compact(skycube_ctx *ctx, const uint32_t *d_rows32, uint32_t *d_membership,
                                   int32_t *d_ext_ids, int64_t *d_offsets, int32_t *d_ids,
                                   int64_t *total_ids, void *stream);

/* Multi-GPU compaction (one call sequence per rank, rank r owning the r-th contiguous
 * range [j_begin, j_end) of S+ tasks, j_begin a multiple of 32, ranges in rank order covering [0, n_ext)):
 *   1. skycube_dev_lattice_count: the rank's per-subspace counts -> d_totals[2^d] (int64, device);
 *   2. the caller gathers every rank's totals into d_all_totals[num_shards][2^d] (e.g. an NCCL all-gather);
 *   3. skycube_dev_lattice_scatter: writes the GLOBAL offsets d_offsets[2^d+1] (nullable) and the rank's ids at
 *      their global positions of `ids` (device memory, or host-mapped pinned memory for a D2H straight into the
 *      caller's result; other ranks' positions are not touched); *total_ids (nullable) = the global id count.
 * d_rows32 is the tiled row buffer of skycube_dev_mdmc (only the rank's range is read).  Between 1 and 3 the
 * context must not run another lattice pass.  With one shard (num_shards = 1, j range = all of S+) this is
 * exactly the lattice of skycube_dev_compact. */
skycube_status skycube_dev_lattice_count(skycube_ctx *ctx, const uint32_t *d_rows32, int64_t j_begin, int64_t j_end,
                                         int64_t *d_totals, void *stream);
skycube_status skycube_dev_lattice_scatter(skycube_ctx *ctx, const uint32_t *d_rows32, int64_t j_begin, int64_t j_end,
                                           const int64_t *d_all_totals, int32_t num_shards, int32_t shard,
                                           int64_t *d_offsets, int32_t *ids, int64_t *total_ids, void *stream);

/* Membership rows by point id of the S+ tasks [j_begin, j_end) (tiled rows of skycube_dev_mdmc), plus zero
 * rows for the points outside S+ whose ids lie in [zero_lo, zero_hi).  `membership` [n][W] is device memory or
 * host-mapped pinned memory; no other row is touched (ranks write disjoint rows of one result). */
skycube_status skycube_dev_membership(skycube_ctx *ctx, const uint32_t *d_rows32, int64_t j_begin, int64_t j_end,
                                      int64_t zero_lo, int64_t zero_hi, uint32_t *membership, void *stream);

/* Partial skycube for the following skycube_dev_mdmc calls (Appendix A.2; see skycube_opts.max_level):
 * 0 = full skycube, d' in [1, 16] = report only |delta| <= d'. */
skycube_status skycube_ctx_set_max_level(skycube_ctx *ctx, int32_t max_level);

/* HashCube (K5) from the complete tiled rows of all S+ points (the d_rows32 of skycube_dev_compact),
 * word length w in [1, 32].  Two calls: with all four output pointers NULL it builds the HashCube in the
 * context's workspace (d_rows32 required) and returns *n_words, *total_keys, *total_ids; then with device
 * buffers d_word_offsets[n_words+1] (int64), d_keys[total_keys] (uint32), d_key_offsets[total_keys+1]
 * (int64), d_ids[total_ids] (int32) it copies the result (same w; d_rows32 ignored).  Layout as
 * skycube_hashcube; ids are point ids. */
skycube_status skycube_dev_hashcube(skycube_ctx *ctx, const uint32_t *d_rows32, uint32_t w, int64_t *d_word_offsets,
                                    uint32_t *d_keys, int64_t *d_key_offsets, int32_t *d_ids, int64_t *n_words,
                                    int64_t *total_keys, int64_t *total_ids, void *stream);

/* Number of kernels launched by this context since creation (for the benchmark's gpu_launches). */
int64_t skycube_ctx_launches(const skycube_ctx *ctx);

/* Work counters accumulated by the context since creation (device-side, read with a sync):
 * out8[0] K1 chunk-corner tests, [1] K1 pair tests, [2] K3 chunk-corner tests, [3] K3 pair tests,
 * [4] K3 misses (pairs that reached Alg. 3 lines 10-12), [5] K3 sub-chunk corner tests, [6..7] reserved (0).  Used by the benchmark's
 * roofline (algorithmic work actually required after pruning). */
skycube_status skycube_ctx_counters(const skycube_ctx *ctx, int64_t *out8);

/* Problem facts after prepare / set_ext: n_ext (0 before set_ext), words per row, and the bit mask of
 * dimensions whose 15-bit codes are injective (exact). Any pointer may be NULL. */
skycube_status skycube_ctx_info(const skycube_ctx *ctx, int64_t *n_ext, uint32_t *words_per_row,
                                uint32_t *exact_mask);

#ifdef __cplusplus
}
#endif

#endif /* SKYCUBE_H */
