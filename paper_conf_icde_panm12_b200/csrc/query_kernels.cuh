// query_kernels.cuh -- argument block of the query kernels (library internal).
#pragma once

#include "common.cuh"

namespace blsh {

struct QueryArgs {
    // sizes
    int64_t nq;
    int d, ds, G, M, B, depth, quantizer, leaf_lo, leaf_hi;
    int probe, T, hstep;
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
};

void upload_e8_roots();
void launch_route_hash(const QueryArgs& a, cudaStream_t s);
void launch_probe_lookup(const QueryArgs& a, cudaStream_t s);
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
};

void launch_items(const int64_t* cnt, int64_t nq, int chunk, int64_t* items, cudaStream_t s);
void launch_shortlist(const ShortlistArgs& a, cudaStream_t s);
void launch_merge(const ShortlistArgs& a, const int32_t* qoor, int64_t* out_ids, float* out_d2,
                  unsigned long long* out_packed, int64_t* out_ncand, cudaStream_t s);

}  // namespace blsh
