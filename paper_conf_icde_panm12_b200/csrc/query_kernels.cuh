// query_kernels.cuh -- argument block of the query kernels (library internal).
#pragma once

#include "common.cuh"
#include "internal.cuh"

namespace blsh {

struct QueryArgs {
    // sizes
    int64_t nq;
    int d, ds, G, M, B, depth, quantizer, leaf_lo, leaf_hi;
    int probe, T, hstep;
    int cperturb;            // probe = 3: bit-perturbed curve keys (R31)
    int msb_min;             // hierarchy = 2: climb threshold on the shared-MSB count (R32; B*M when 0)
    int64_t rec_tau;         // probe = 2, T > 241: second-ring probes only while |A| < rec_tau (R33; 0 = all)
    // queries
    const float* Q;          // [nq][ds]
    // tree + params
    const float* dirs;
    const float* mu;
    const float* theta;
    const int32_t* ntype;
    const float* A;
    const float* bvec;
    const float* Wl;
    // table
    const Key128* ukey;
    const uint32_t* uoff;
    const int64_t* leaf_u;
    // per-query outputs
    int32_t* qleaf;
    float* qt;
    int32_t* qcode;
    int32_t* qoor;           // bit0: home code out of range, bit1: leaf not owned
    Key128* qkey;
    Key128* pkey;            // nullable (keep_stages)
    int32_t* pvalid;         // nullable
    uint2* ivl;              // [nq][T+1]
    int64_t* base;
    int64_t* cnt;
    int32_t* level;          // nullable
    uint32_t* lperm;         // [nq] queries grouped by leaf (a1 -> a2)
    int32_t* lcnt;           // [2G] leaf counts, scatter cursors
    // short-list screen's compact table (resid.cu)
    int dr;
    const void* Rh;          // fp16 rows in swizzled 8-row atoms (resid.cu)
    int64_t natom;           // atoms of the table
    const float4* rconst;
    const uint32_t* rgrp;    // [n_owned] anchor group of every table row
    const float* anc;        // [anchor blocks][dr]
};

void upload_e8_roots();
int launch_route_hash(const QueryArgs& a, cudaStream_t s);   // returns kernels launched
void launch_probe_lookup(const QueryArgs& a, cudaStream_t s);
void launch_msb_climb(const QueryArgs& a, cudaStream_t s);
int launch_route_group(const QueryArgs& a, cudaStream_t s);
void launch_gather_rows(const float* Q, int ds, const uint32_t* idx, int64_t n, float* out, cudaStream_t s);
void launch_shard_outputs(const uint32_t* idx, int64_t nq, int64_t n, int k, const int64_t* ids_c, const float* d2_c,
                          const unsigned long long* pk_c, const int64_t* nc_c, int64_t* ids, float* d2,
                          unsigned long long* pk, int64_t* nc, cudaStream_t s);
// a2 only (queries already routed and grouped by leaf in a.lperm): hash with a.A / a.bvec
void launch_hash(const QueryArgs& a, cudaStream_t s);
// a2 of several hash tables in one launch (tables 1..L-1 of an L-table index)
constexpr int kMaxTables = 64;
struct HashTables {
    int n;
    const float* A[kMaxTables];
    const float* b[kMaxTables];
    float* qt[kMaxTables];
    int32_t* qcode[kMaxTables];
    int32_t* qoor[kMaxTables];
    Key128* qkey[kMaxTables];
};
void launch_hash_tables(const QueryArgs& a, const HashTables& ht, cudaStream_t s);

// L > 1 tables (tables.cu): raw[q] = sum over tables of |A0_l(q)|, then the
// deduplicated union of the L tables' intervals as ascending table-0 positions.
struct UnionArgs {
    int64_t nq;
    int L, T;
    const int32_t* qleaf;
    const int32_t* qoor;          // table 0's flags (bit 1: leaf not owned)
    const uint2* const* ivl;      // [L] device pointers to [nq][T+1]
    const int64_t* const* cnt;    // [L] device pointers to [nq]
    const uint32_t* const* pos;   // [L] table-l position -> table-0 position ([0] = identity)
    const int64_t* leaf_pos;      // [G+1]
    const int64_t* raw_off;       // [nq+1]
    int64_t* raw;                 // [nq]
    uint32_t* list;               // [raw_off[nq]]
    int64_t* out_cnt;             // [nq] |A(q)|
    // E8 hierarchy node (NULL hlevel: none): buckets [hs, he) of level hlevel's order
    const int32_t* hlevel;
    const int64_t* hs;
    const int64_t* he;
    const int64_t* hrows;
    const uint32_t* const* lv_bu; // [kE8Levels + 1] bucket of each position of level j's order
    const uint32_t* uoff;         // bucket row offsets (primary table)
};

// E8 code hierarchy (e8hier.cu, R27)
constexpr int kE8Levels = 32;
struct E8WidenArgs {
    int64_t nq;
    int M, B;                     // M = 8 or 16 (E8 blocks)
    const int32_t* qleaf;
    const int32_t* qoor;
    const int32_t* qcode;         // [nq][M] doubled home codes
    const int64_t* base;          // |A0(q)|
    const Key128* ukey;           // level 0 keys (the table)
    const uint32_t* uoff;
    const int64_t* leaf_u;
    const int32_t* root;          // [G] first level at which a leaf's buckets share one code
    const Key128* const* lv_key;  // [kE8Levels + 1]
    const int64_t* const* lv_cum; // [kE8Levels + 1] running rows of level j's order
    int32_t* hlevel;              // out: level (kE8Levels + 1 = whole leaf; 0 = not widened)
    int64_t* hs;
    int64_t* he;
    int64_t* hrows;
};
void launch_e8_widen(const E8WidenArgs& w, const int64_t* tau, int64_t min_cand, cudaStream_t s);
void launch_raw_counts(const UnionArgs& u, cudaStream_t s);
void launch_union_tables(const UnionArgs& u, int64_t max_leaf_rows, cudaStream_t s);
void launch_median(const int64_t* base, int64_t nq, int64_t* tau, cudaStream_t s);
void launch_widen(const QueryArgs& a, const int64_t* tau, int64_t min_cand, cudaStream_t s);

struct ShortlistArgs {
    int64_t nq, n_items;
    int d, ds, T, k, chunk;
    const float* Q;          // [nq][ds]
    const float* Xp;         // [n_owned][ds]
    const uint32_t* perm;
    const uint2* ivl;        // [nq][T+1]
    const int64_t* cnt;
    const int64_t* item_off; // [nq+1]
    unsigned long long* partials;   // [n_items][k]
    const int64_t* cand_off;        // [nq+1] (large k)
    unsigned long long* cand_keys;  // [total] non-NULL: emit every candidate key (large k)
    const uint32_t* list;           // non-NULL (L > 1): deduplicated candidate positions per query
    const int64_t* list_off;        // [nq+1] start of each query's list
    const int64_t* n_items_dev;     // non-NULL: the item count lives on the device (n_items is then an upper
                                    // bound for the grid; small batches plan without a host round trip)
};

// query-tiled short-list (shortlist_tiled.cu)
// 0: warp short-list, 1: SIMT query-tiled, 2: tensor-core screened query-tiled.  The TC
// kernel is the default where it applies (k <= 32, d_stride a multiple of 64 and <= 512);
// BLSH_SHORTLIST=warp|simt forces the others.
int shortlist_kind(int64_t nq, int ds, int dr, int T, int k);
int64_t small_batch_limit();   // batches up to this size take the warp short-list
void sort_queries(const QueryArgs& a, SortBufs& sb, uint32_t* qorder, cudaStream_t s, int* launches);
int64_t plan_tiles(const QueryArgs& a, const uint32_t* qorder, DevBuf& tilebuf, ScanTemp& scan, cudaStream_t s,
                   int* launches);
void run_tiled_shortlist(const QueryArgs& a, const uint32_t* qorder, int k, DevBuf& segbuf, DevBuf& tilebuf,
                         DevBuf& rowbuf,
                         DevBuf& partials, DevBuf& keybuf, ScanTemp& scan, int64_t* out_ids, float* out_d2,
                         unsigned long long* out_packed, int64_t* out_ncand, const float* Xp, const uint32_t* perm,
                         cudaStream_t s, int* launches, int64_t* n_items_out, int* chr_out, int64_t* rows_out,
                         cudaEvent_t ev_sl0, cudaEvent_t ev_mid, cudaEvent_t ev_sl1, int64_t* pairs_out,
                         int64_t* kept_out, double* qload_rows_out, int kind, int64_t ntiles,
                         int64_t* kslots_out, int* screen_kind_out);

void launch_items(const int64_t* cnt, int64_t nq, int chunk, int64_t* items, cudaStream_t s);
void launch_shortlist(const ShortlistArgs& a, cudaStream_t s);
void launch_select(const unsigned long long* cand_keys, const int64_t* cand_off, int64_t nq, int k,
                   const int32_t* qoor, const int64_t* cnt, int64_t* out_ids, float* out_d2,
                   unsigned long long* out_packed, int64_t* out_ncand, cudaStream_t s);
void launch_merge(const ShortlistArgs& a, const int32_t* qoor, int64_t* out_ids, float* out_d2,
                  unsigned long long* out_packed, int64_t* out_ncand, cudaStream_t s);

}  // namespace blsh
