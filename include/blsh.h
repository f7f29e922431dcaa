/*
 * include/blsh.h -- C ABI of the B200-native Bi-level LSH query hot path.
 *
 * Bi-level LSH (Pan & Manocha, ICDE 2012; "P:n" = line n of the paper text):
 * a first-level RP-tree partitions the data into subgroups, each
 * subgroup gets its own E2LSH table with M projections of width W (P:41-43,
 * P:121-127) stored as one linear array sorted by the bi-level code
 * (leaf, Morton(H(v))).  A query is routed to its leaf,
 * hashed, its buckets are probed (standard, multiprobe P:247, E8 lattice
 * P:138-147, optional Morton-prefix widening P:132 / P:249-251) and the
 * short-list search ranks the candidates by exact distance.
 *
 * Conventions for every call
 *  - Pointers may be CUDA device pointers or host pointers (pageable or
 *    pinned); the library detects which with cudaPointerGetAttributes and
 *    stages host buffers through device memory on `stream`.  Device pointers
 *    must be 16-byte aligned for X and Q.
 *  - All arrays are C-contiguous, row-major.  Floating point inputs are fp32.
 *  - Calls are ordered on the CUDA stream given in the params struct (NULL =
 *    legacy default stream).  blsh_build / blsh_query return after the stream
 *    work they enqueued has completed (they synchronise `stream`), so host
 *    outputs are valid on return.
 *  - Every call returns a blsh_status and never throws across the ABI.  On
 *    failure blsh_last_error() returns a thread-local message; outputs are
 *    unspecified and nothing is leaked.
 *  - Inputs with NaN/Inf are undefined behaviour.
 *  - The index owns all of its device memory until blsh_free.
 * Readings of the paper that the arithmetic follows are listed in DESIGN.md
 * (R1..R24); the library and the CPU oracle implement them independently.
 */
#ifndef BLSH_H
#define BLSH_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct blsh_index blsh_index;       /* opaque, owned by the library */

typedef enum {
    BLSH_OK = 0,
    BLSH_ERR_INVALID = 1,      /* bad argument (checked before any device work)          */
    BLSH_ERR_OOM = 2,          /* device allocation failed                                */
    BLSH_ERR_CUDA = 3,         /* CUDA runtime / launch error                             */
    BLSH_ERR_RANGE = 4,        /* a data point's code leaves the B-bit Morton range (R9)  */
    BLSH_ERR_UNSUPPORTED = 5   /* valid request outside what this build implements        */
} blsh_status;

/* Build parameters.  Defaults: blsh_build_params_default(). */
typedef struct {
    int32_t n_leaves;       /* G: RP-tree leaves, power of two in [1, 4096] (R8); 1 = standard LSH */
    int32_t rp_rule;        /* 0 = RP-tree mean (default), 1 = RP-tree max                    */
    double  rp_mean_c;      /* c of the mean-rule test Delta^2 <= c * Delta_A^2 (R4; default 10)           */
    double  rp_max_jitter;  /* j of the max-rule jitter (R4; default 0)                                     */
    int32_t ek_iters;       /* m of the approximate diameter (R6; default 40)                        */
    int32_t M;              /* hash dimension, 1..16; exactly 8 for E8                               */
    int32_t quantizer;      /* 0 = Z^M floor (Eq. 2), 1 = E8 DECODE (Eq. 6)                                 */
    float   W;              /* bucket width > 0                                                       */
    const float* W_leaf;    /* optional HOST array [G] of per-leaf widths (R3); NULL = W everywhere  */
    uint64_t seed;          /* seed of the counter-based generator (R2)                                     */
    int32_t rank, world;    /* shard: this index keeps leaves [rank*G/world, (rank+1)*G/world) (default 0,1),
                               or the leaf_split ranges below                                                */
    void*   stream;         /* cudaStream_t                                                                 */
    int32_t keep_stages;    /* 1 = keep per-point leaf/code/key for blsh_export (parity tests)              */
    int32_t n_tables;       /* L hash tables per leaf, 1..64 ("L hash tables ... each constructed
                               independently with different dim-M hash functions"; default 1).  Table l
                               draws its own (a, b) (R2 streams (1, l, g), (2, l, g)); the RP-tree, W and
                               the stored rows are shared.  A query's candidate set is the union of its
                               probed buckets over the L tables, deduplicated (R24).  L > 1 needs every
                               owned leaf to hold <= 1,600,000 points (the per-query dedup bitmap lives
                               in shared memory) and excludes the Morton hierarchy.                      */
    const int32_t* leaf_split; /* optional HOST array [world+1]: rank r keeps leaves [leaf_split[r],
                               leaf_split[r+1]) -- a load-aware contiguous assignment (SURVEY §8(e):
                               query skew across leaves); leaf_split[0] = 0, leaf_split[world] = G,
                               non-decreasing, identical on every rank.  NULL = G/world leaves each
                               (then world must divide G).                                                */
    int32_t W_rule;         /* 0 = W (or W_leaf) for every leaf; 1 = per-leaf width adapted to the leaf's
                               spread ("different LSH parameters (e.g. bucket size W) that are optimal
                               for each cell"; R29): W_g = fp32(W * sqrt(D_g / D_med)), D_g = Delta_A^2 of
                               leaf g (R7), D_med = the lower median of D over the leaves; W_g = W for leaves
                               with D_g = 0.  Exported as BLSH_EX_W.  Excludes W_leaf.                       */
} blsh_build_params;

/* Query parameters.  Defaults: blsh_query_params_default(). */
typedef struct {
    int32_t probe;          /* 0 standard (T = 1), 1 multiprobe on Z^M (R11), 2 lattice on E8,
                               3 Morton-curve neighbours on Z^M (R25): the T buckets around the
                               insertion position of the home key in the leaf's sorted keys (after, before,
                               alternating)                                                                    */
    int32_t n_probes;       /* T >= 1 including the home bucket; <= 3^M (M <= 10), <= 256 (Morton curve) or
                               <= 256 (E8: home, the 240 roots, then probes 242..256 from the second ring of
                               recursive probing, R26)                                                */
    int32_t hierarchy;      /* 1 = Morton-prefix widening until |R| >= tau (Eq. 7-8, R17) on a Z^M index,
                               the E8 code hierarchy (R27) on an E8 index; 2 = P:132's shared-MSB
                               climb (R32, Z^M): a query whose home key shares fewer than msb_min leading
                               bits with the keys before/after its insertion position also takes the leaf's
                               buckets that share those bits with it                                         */
    int32_t hier_step_bits; /* key bits cleared per widening step: 0 = M (one Eq. 8 level), or 1..M           */
    int64_t min_cand;       /* tau (R18); 0 = lower median of the base counts of this batch.         
                               probe = 2 (E8, M = 8) with hierarchy = 0 and min_cand > 0: recursive lattice
                               probing ("if the number of candidates computed is not enough, we
                               recursively probe the adjacent buckets of the 240 probed buckets", R33): the
                               second-ring probes 241..n_probes-1 are taken in order only while the probes
                               before them hold < min_cand candidates (not taken: Q_PVALID 0); needs L = 1  */
    void*   stream;         /* cudaStream_t                                                                   */
    int32_t keep_stages;    /* 1 = keep per-query stages of this call for blsh_export                         */
    int32_t timing;         /* 1 = record per-stage CUDA-event times into blsh_last_stats                     */
    const int64_t* global_base; /* optional DEVICE array [nq]: |A0(q)| of every query of the batch summed over
                               the shards (blsh_query_base_counts on each rank + a sum all-reduce).  With
                               hierarchy = 1 and min_cand = 0, tau = its lower median (R18: P:249's "median
                               over a set of queries" taken over the whole sharded batch, so a sharded index
                               widens exactly like one GPU).  NULL = this call's own counts; must be non-NULL
                               for that case when world > 1.  Read on `stream`; owned by the caller.          */
    int32_t curve_perturb;  /* probe = 3 only, 0..M: P:132's bit-perturbed repeats of the curve search (R31):
                               keys = the home key and the home key with bit 0 of its curve_perturb nearest
                               coordinates flipped; probe j searches around key j mod (curve_perturb + 1);
                               an already probed bucket is an empty probe                                     */
    int32_t msb_min;        /* hierarchy = 2: climb when the shared-MSB count s* < msb_min; 0 = B*M (every
                               query whose home bucket is empty)                                              */
} blsh_query_params;

void blsh_build_params_default(blsh_build_params* p);
void blsh_query_params_default(blsh_query_params* p);

/* b1-b4: parameters, RP-tree, data hash, table.
 *   X [n x d] fp32 (device or host).  d in [1, 1024].  n in [0, 2^31).
 *   The library copies X into its own layout; X may be freed after return.
 *   *out receives the index, or NULL on failure. */
blsh_status blsh_build(const float* X, int64_t n, int32_t d, const blsh_build_params* p,
                       blsh_index** out);

/* a1-a5: route, hash, probe, look up, (widen), short-list.
 *   Q         [nq x d] fp32 queries (device or host)
 *   k         neighbours, 1..1024 (k > 1024 -> BLSH_ERR_UNSUPPORTED).  k <= 64 keeps
 *             per-warp register top-k lists; 64 < k <= 1024 (the paper evaluates
 *             k = 500) emits every candidate's packed (d^2, id) key to a
 *             workspace of 8 B per candidate and selects per query (radix select);
 *             both give the k smallest by (d^2, id).
 *   out_ids   [nq x k] int64 original row ids of X, ascending (d^2, id); -1 = padding
 *   out_dist2 [nq x k] fp32 squared L2 distances (fp32, direct form, R22); +inf = padding
 *   out_ncand [nq] int64 |A(q)| (may be NULL)
 * A query whose leaf is not owned by this shard returns only padding and 0. */
blsh_status blsh_query(const blsh_index* idx, const float* Q, int64_t nq, int32_t k,
                       const blsh_query_params* p, int64_t* out_ids, float* out_dist2,
                       int64_t* out_ncand);

/* a1-a5 over a stream of n_batches independent HOST batches (serving form of
 * blsh_query; the same problem statement, per batch): batch b is
 * Q[b] [nq x d] fp32 in host memory, its answers go to out_ids[b] [nq x k],
 * out_dist2[b] [nq x k] and out_ncand[b] [nq] (may be NULL) in host memory.
 * Results equal n_batches separate blsh_query calls (every batch-level
 * statistic, e.g. the hierarchy's median tau R18, is taken per batch).  The
 * library uploads batch b+1 and downloads batch b-1 on its own copy stream
 * while batch b is searched on p->stream (two device staging buffers for the
 * queries and for the answers), so with page-locked host buffers the copies
 * overlap the search.  Pointers in the arrays may repeat (e.g. one host batch
 * searched n_batches times); an output buffer is overwritten in batch order.
 * Host buffers only (BLSH_ERR_INVALID for device pointers); returns after
 * every copy has completed. */
blsh_status blsh_query_pipelined(const blsh_index* idx, int32_t n_batches, const float* const* Q,
                                 int64_t nq, int32_t k, const blsh_query_params* p,
                                 int64_t* const* out_ids, float* const* out_dist2,
                                 int64_t* const* out_ncand);

/* Multi-GPU form of blsh_query: each row is k packed u64 entries
 * (float_bits(d^2) << 32) | id32, ascending; padding = 0x7F800000FFFFFFFF.
 * For d^2 >= 0 integer order equals (d^2, id) order.  Requires n < 2^32. */
blsh_status blsh_query_packed(const blsh_index* idx, const float* Q, int64_t nq, int32_t k,
                              const blsh_query_params* p, uint64_t* out_packed,
                              int64_t* out_ncand);

/* a1-a4 only (route, hash, probe, look up; no widening, no short-list): the
 * base candidate count |A0(q)| of every query (the count the hierarchy's
 * threshold is a median of), 0 for queries whose leaf another shard owns.
 *   Q        [nq x d] fp32 (device or host)
 *   out_base [nq] int64 (device or host)
 * On a sharded index the sum over ranks of out_base is the single-GPU base
 * count of every query; pass it as p->global_base to blsh_query(_packed). */
blsh_status blsh_query_base_counts(const blsh_index* idx, const float* Q, int64_t nq,
                                   const blsh_query_params* p, int64_t* out_base);

/* a6: merge n_lists per-rank packed lists (e.g. the output of an NCCL
 * all-gather, layout [n_lists][nq][k]) into the k smallest per query.
 * packed is a device pointer; outputs device or host.  k in 1..1024. */
blsh_status blsh_merge_topk(const uint64_t* packed, int32_t n_lists, int64_t nq, int32_t k,
                            int64_t* out_ids, float* out_dist2, void* stream);

/* Export build artefacts / last-query stages into HOST memory dst (cap bytes).
 * *needed (may be NULL) receives the byte size; if dst is NULL or cap is too
 * small the call returns BLSH_ERR_INVALID after setting *needed. */
typedef enum {
    BLSH_EX_A = 0,          /* float [G][M][d]  projection vectors a_i per leaf      */
    BLSH_EX_B = 1,          /* float [G][M]     offsets b_i per leaf                          */
    BLSH_EX_W = 2,          /* float [G]        widths                                        */
    BLSH_EX_DIRS = 3,       /* float [G-1][d]   RP directions                          */
    BLSH_EX_MU = 4,         /* float [G-1][d]   node means (mean rule)                        */
    BLSH_EX_THETA = 5,      /* float [G-1]      split thresholds                              */
    BLSH_EX_NTYPE = 6,      /* int32 [G-1]      0 hyperplane, 1 sphere                        */
    BLSH_EX_DIAM2 = 7,      /* double [G-1]     diameter estimate^2 (R6)                      */
    BLSH_EX_DA2 = 8,        /* double [G-1]     Delta_A^2 (R7)                                */
    BLSH_EX_PERM = 10,      /* int64 [n_owned]  table position -> original id                 */
    BLSH_EX_UKEY = 11,      /* uint64 [nu][2]   bucket keys (hi, lo)                          */
    BLSH_EX_ULEAF = 12,     /* int32 [nu]       bucket leaf                                   */
    BLSH_EX_UOFF = 13,      /* int64 [nu+1]     bucket start positions                        */
    BLSH_EX_LEAF_U = 14,    /* int64 [G+1]      first bucket of each leaf                     */
    BLSH_EX_RGRP = 15,      /* int32 [n_owned]  screen anchor group of every table row (resid.cu) */
    BLSH_EX_GSTART = 16,    /* int64 [groups+1] first table row of every anchor group          */
    BLSH_EX_POINT_LEAF = 20,/* int32 [n]        leaf of every point (keep_stages)             */
    BLSH_EX_POINT_CODE = 21,/* int32 [n][M]     code (Z^M floor / doubled E8), owned points   */
    BLSH_EX_POINT_KEY = 22, /* uint64 [n][2]    Morton key (hi, lo), owned points             */
    BLSH_EX_Q_LEAF = 30,    /* int32 [nq]       last query: leaf                              */
    BLSH_EX_Q_T = 31,       /* float [nq][M]    projections t                                 */
    BLSH_EX_Q_CODE = 32,    /* int32 [nq][M]    clamped home code                             */
    BLSH_EX_Q_OOR = 33,     /* int32 [nq]       1 = home code outside the Morton range; 5 = non-finite
                               projection (NaN/Inf query, R30): no probes, no candidates      */
    BLSH_EX_Q_KEY = 34,     /* uint64 [nq][2]   home key (0 when out of range)                */
    BLSH_EX_Q_PKEY = 35,    /* uint64 [nq][T][2] probe keys in probe order (0 = invalid)      */
    BLSH_EX_Q_PVALID = 36,  /* int32 [nq][T]    probe key inside the range                    */
    BLSH_EX_Q_BASE = 37,    /* int64 [nq]       |A0| before widening                          */
    BLSH_EX_Q_LEVEL = 38,   /* int32 [nq]       key bits cleared by the hierarchy (0 = none)  */
    BLSH_EX_Q_TAU = 39,     /* int64 [1]        threshold used                                */
    BLSH_EX_Q_INTERVALS = 40,/* int64 [nq][T+1][2] candidate intervals [start, end) in table positions */
    BLSH_EX_Q_CAND_OFF = 41,/* int64 [nq+1]     list path (L > 1 or E8 hierarchy): offsets into Q_CAND      */
    BLSH_EX_Q_CAND = 42     /* int64 [sum|A(q)|] list path: candidate ids of every query, ascending           */
} blsh_export_what;
/* Table l of an L-table index (n_tables > 1): what = BLSH_EX_TABLE(l, item) for
 * the per-table items A, B, PERM (original ids in table-l order), UKEY, ULEAF,
 * UOFF (table-l positions), LEAF_U and the per-table query stages Q_T .. Q_BASE
 * (Q_BASE = |A0_l(q)| of table l) and Q_INTERVALS (table-l positions).  l = 0
 * is the primary table (plain item codes). */
#define BLSH_EX_TABLE(l, item) ((int32_t)(((l) << 8) | (item)))

blsh_status blsh_export(const blsh_index* idx, int32_t what, void* dst, size_t cap,
                        size_t* needed);

typedef struct {
    int64_t n, n_owned, nu;
    int32_t d, d_stride, G, M, B, quantizer;
    int32_t leaf_lo, leaf_hi;   /* owned leaves [leaf_lo, leaf_hi) */
    int64_t device_bytes;       /* persistent device memory held by the index */
    double  build_ms;           /* wall time of blsh_build                      */
    int32_t n_tables;           /* L */
    int32_t pad_;
} blsh_info;

blsh_status blsh_index_info(const blsh_index* idx, blsh_info* out);

/* Statistics of the last blsh_query / blsh_query_packed on this index. */
typedef struct {
    int64_t nq, n_active, total_cand, n_items, tau;
    int32_t chunk, launches;          /* candidates (rows) per work item; kernels launched by the call */
    double  shortlist_bytes;          /* algorithmic bytes of the short-list: sum|A(q)|*d*4 + 4/candidate + outputs */
    float   ms_route_hash, ms_probe, ms_plan, ms_shortlist, ms_merge, ms_total;  /* timing = 1 */
    int32_t tiled;                    /* 1 = query-tiled short-list (rows shared across a tile of 32 queries) */
    int32_t pad_;
    int64_t union_rows;               /* tiled: rows streamed from HBM (sum over tiles of the candidate union) */
    int64_t pairs_scored;             /* (row, query) distance evaluations actually performed */
    double  shortlist_flops;          /* algorithmic flops: 3*d per (query, candidate) pair */
    float   ms_screen, ms_rescore;    /* tiled: the streaming kernel alone; TC: the exact rescoring kernel (timing = 1) */
    double  union_bytes;              /* tiled: algorithmic bytes of the streaming kernel: union rows x (4 d_stride + 8)
                                         + the tile queries each work item loads (4 d_stride per query)              */
    int64_t pairs_kept;               /* TC: (row, query) pairs that passed the running screen and were buffered   */
    int64_t k_slots;                  /* fp16 screen: (tile, anchor block) pairs of the K table                    */
    int32_t screen_row_bytes;         /* bytes per union row the screen kernel reads (rows + metadata)            */
    int32_t screen_kind;              /* 0 none, 1 fp16 compact-table screen (k_screen_f16), 2 TF32 (k_shortlist_tc) */
} blsh_stats;

blsh_status blsh_last_stats(const blsh_index* idx, blsh_stats* out);

void        blsh_free(blsh_index* idx);     /* NULL-safe */
const char* blsh_last_error(void);          /* thread-local message of the last failure */

#ifdef __cplusplus
}
#endif
#endif /* BLSH_H */
