// internal.cuh -- library-internal declarations (index layout, launchers).
#pragma once

#include <cuda_runtime.h>

#include <cstdint>
#include <memory>
#include <stdexcept>
#include <string>
#include <vector>

#include "../../include/blsh.h"
#include "common.cuh"

namespace blsh {

// Error carrying a blsh_status; converted at the ABI boundary.
struct Error : std::runtime_error {
    blsh_status code;
    Error(blsh_status c, const std::string& m) : std::runtime_error(m), code(c) {}
};

#define BLSH_CUDA(expr)                                                                      \
    do {                                                                                     \
        cudaError_t e__ = (expr);                                                            \
        if (e__ != cudaSuccess)                                                              \
            throw ::blsh::Error(e__ == cudaErrorMemoryAllocation ? BLSH_ERR_OOM : BLSH_ERR_CUDA, \
                                std::string(#expr) + ": " + cudaGetErrorString(e__) + " @" + \
                                __FILE__ + ":" + std::to_string(__LINE__));                  \
    } while (0)

#define BLSH_LAUNCH_CHECK() BLSH_CUDA(cudaGetLastError())

// Device buffer owned by RAII.
struct DevBuf {
    void* p = nullptr;
    size_t bytes = 0;
    DevBuf() = default;
    DevBuf(const DevBuf&) = delete;
    DevBuf& operator=(const DevBuf&) = delete;
    ~DevBuf() { release(); }
    void release() {
        if (p) cudaFree(p);
        p = nullptr;
        bytes = 0;
    }
    void alloc(size_t b) {
        release();
        if (b == 0) b = 16;
        BLSH_CUDA(cudaMalloc(&p, b));
        bytes = b;
    }
    void ensure(size_t b) {   // grow-only, contents not preserved
        if (b > bytes) alloc(b + b / 4);
    }
    template <typename T> T* as() const { return reinterpret_cast<T*>(p); }
};

// Bump allocator over a DevBuf (alignment 256 B).
struct Arena {
    char* base = nullptr;
    size_t off = 0, cap = 0;
    template <typename T> T* take(size_t count) {
        size_t b = (count * sizeof(T) + 255) & ~size_t(255);
        if (off + b > cap) throw Error(BLSH_ERR_INVALID, "internal arena overflow");
        T* r = reinterpret_cast<T*>(base + off);
        off += b;
        return r;
    }
    static size_t need(size_t count, size_t elem) { return (count * elem + 255) & ~size_t(255); }
};

// Temp storage of the device scan.
struct ScanTemp {
    DevBuf blocks;
};

// ---- primitives (scan.cu, sort.cu) ------------------------------------------
// out[i] = sum_{j<i} in[j] for i in [0, n]; out has n+1 entries.
void scan_exclusive_i64(const int64_t* in, int64_t* out, int64_t n, ScanTemp& t, cudaStream_t s);
void scan_exclusive_u8(const uint8_t* in, int64_t* out, int64_t n, ScanTemp& t, cudaStream_t s);

struct SortBufs {
    DevBuf hi[2], lo[2], leaf[2], id[2], hist, off, stats;
    ScanTemp scan;
};
// Stable LSD radix sort of (leaf, hi, lo) with payload id; result in buffer index returned.
int radix_sort_entries(SortBufs& b, int64_t n, cudaStream_t s, int* passes_done);

// ---- index -----------------------------------------------------------------
struct QueryWork {
    DevBuf arena;      // per-call carve-outs
    DevBuf partials;   // per-item partial top-k lists
    DevBuf host_stage; // device staging for host outputs
    DevBuf segbuf, tilebuf;   // tiled short-list: per-tile segments, tile arrays
    DevBuf keybuf;            // tiled short-list, large k: per-query segments of exact (d^2, id) keys
    DevBuf rowbuf;            // tiled short-list: per-union-row entries, K table, item rows
    SortBufs qsort;           // query sort by (leaf, key)
    ScanTemp scan;
    int64_t nq = 0;
    int T = 0, k = 0;
    // carved pointers of the last call
    float* Qd = nullptr;
    int32_t* qleaf = nullptr;
    float* qt = nullptr;
    int32_t* qcode = nullptr;
    int32_t* qoor = nullptr;
    Key128* qkey = nullptr;
    Key128* pkey = nullptr;
    int32_t* pvalid = nullptr;
    uint2* ivl = nullptr;      // [nq][T+1] (start, end)
    int64_t* base = nullptr;
    int64_t* cnt = nullptr;
    int32_t* level = nullptr;
    int64_t* item_off = nullptr;  // [nq+1]
    int64_t* tau = nullptr;
    int64_t* ncand_dev = nullptr;
    int64_t* misc = nullptr;      // small scalars
    // L > 1 tables: per-table a2-a4 stages (tq[0] aliases the fields above)
    struct TableQuery {
        float* qt; int32_t* qcode; int32_t* qoor; Key128* qkey; Key128* pkey; int32_t* pvalid;
        uint2* ivl; int64_t* base; int64_t* cnt;
    };
    std::vector<TableQuery> tq;
    DevBuf listbuf;               // deduplicated candidate positions (u32), at raw_off[q]
    DevBuf sh_qfull, sh_buf;      // sharded index: the whole batch on the device; routing + compact batch
    int64_t* raw_off = nullptr;   // [nq+1] scan of the per-query sums of the table counts
    bool list_valid = false;      // the last query built candidate lists (listbuf / raw_off / cnt)
    // side stream: the query sort and tile formation run while a3/a4 run on the caller's stream
    ScanTemp scan2;
    cudaStream_t side = nullptr;
    cudaEvent_t ev_fork = nullptr, ev_join = nullptr;
    int64_t* host_scalars = nullptr;   // pinned [3]: plan statistics and tau, read back with the answers
    // small batches: the whole call captured once per shape into a CUDA graph (api.cu, query_graph)
    struct GraphEntry {
        int64_t nq, min_cand;
        int k, T, probe, hierarchy, hstep, cperturb, msb_min;
        const void* bufs[6];
        size_t sizes[6];
        cudaGraphExec_t exec;
        blsh_stats stats;
    };
    std::vector<GraphEntry> graphs;
    DevBuf g_q, g_out;                 // the graphs' query batch and answers
    cudaStream_t cap = nullptr;        // capture stream
    // blsh_query_pipelined: double-buffered query uploads / answer downloads on a copy stream
    DevBuf pl_q[2], pl_out[2];
    cudaStream_t copy = nullptr;
    cudaEvent_t pl_up[2] = {nullptr, nullptr}, pl_free[2] = {nullptr, nullptr}, pl_dl[2] = {nullptr, nullptr};
    QueryWork() = default;
    QueryWork(const QueryWork&) = delete;
    QueryWork& operator=(const QueryWork&) = delete;
    ~QueryWork() {
        if (ev_fork) cudaEventDestroy(ev_fork);
        if (ev_join) cudaEventDestroy(ev_join);
        if (side) cudaStreamDestroy(side);
        for (int i = 0; i < 2; ++i) {
            if (pl_up[i]) cudaEventDestroy(pl_up[i]);
            if (pl_free[i]) cudaEventDestroy(pl_free[i]);
            if (pl_dl[i]) cudaEventDestroy(pl_dl[i]);
        }
        if (copy) cudaStreamDestroy(copy);
        for (auto& g : graphs)
            if (g.exec) cudaGraphExecDestroy(g.exec);
        if (cap) cudaStreamDestroy(cap);
        if (host_scalars) cudaFreeHost(host_scalars);
    }
};

// Hash table l >= 1 of an L-table index.  Table 0 is the primary
// table (blsh_index fields); the rows of X are stored once, in table-0 order,
// and table l refers to them through pos (table-l position -> table-0 position).
struct ExtraTable {
    DevBuf A, b;          // [G][M][d], [G][M] this table's (a, b) (R2 streams (1, l, g), (2, l, g))
    DevBuf ukey;          // [nu] Key128
    DevBuf uleaf;         // [nu] int32
    DevBuf uoff;          // [nu+1] uint32 (table-l positions)
    DevBuf leaf_u;        // [G+1] int64
    DevBuf pos;           // [n_owned] uint32 table-0 position of the row at table-l position i
    DevBuf perm;          // [n_owned] uint32 original ids in table-l order (export / parity)
    int64_t nu = 0;
    std::vector<float> A_h, b_h;
    std::vector<int64_t> leaf_u_h;
};

}  // namespace blsh

struct blsh_index {
    // metadata
    int64_t n = 0, n_owned = 0, nu = 0;
    int d = 0, ds = 0, G = 1, M = 8, B = 16, quantizer = 0, depth = 0;
    int leaf_lo = 0, leaf_hi = 1, rank = 0, world = 1;
    int rp_rule = 0, ek_iters = 40;
    double rp_mean_c = 10.0, rp_max_jitter = 0.0;
    uint64_t seed = 0;
    double build_ms = 0.0;
    // host copies (export)
    std::vector<float> A_h, b_h, W_h, dirs_h, mu_h, theta_h;
    std::vector<int32_t> ntype_h;
    std::vector<double> diam2_h, da2_h, jit_h;
    std::vector<double> leaf_da2_h;    // [G] W rule 1: Delta_A^2 of every leaf (R29)
    std::vector<int64_t> leaf_u_h;     // [G+1]
    // device: parameters and tree
    blsh::DevBuf A, b, W, dirs, mu, theta, ntype;
    // device: table
    blsh::DevBuf Xp;      // [n_owned][ds] fp32 rows in table order
    blsh::DevBuf perm;    // [n_owned] uint32 original ids
    blsh::DevBuf ukey;    // [nu] Key128
    blsh::DevBuf uleaf;   // [nu] int32
    blsh::DevBuf uoff;    // [nu+1] uint32
    blsh::DevBuf leaf_u;  // [G+1] int64
    // device: the short-list screen's compact rows (resid.cu): anchor groups of consecutive buckets
    int dr = 0;                 // fp16 columns per row (ds rounded up to 64)
    int64_t nanchor = 0;        // anchor groups
    float anchor_tau2 = 0.f;    // grouping threshold (squared distance between consecutive bucket means)
    blsh::DevBuf anc;           // [nanchor][dr] fp32 anchors a_g
    blsh::DevBuf gstart;        // [nanchor+1] int64 first table row of every group
    blsh::DevBuf rgrp;          // [n_owned] uint32 group of every table row
    blsh::DevBuf Rh;            // fp16 residuals r = (x - a_g) / s_g in swizzled 8-row atoms (resid.cu)
    blsh::DevBuf rconst;        // [atoms * 8] float4 (|s_g r|^2, s_g, |s_g r|, G); zero for padding rows
    // L > 1 hash tables
    int L = 1;
    std::vector<std::unique_ptr<blsh::ExtraTable>> xt;   // tables 1..L-1
    std::vector<int64_t> leaf_pos_h;   // [G+1] first owned table position of each leaf (clamped)
    blsh::DevBuf leaf_pos;             // device copy
    blsh::DevBuf tab_pos;              // [L] const uint32_t* (pos of table l; [0] = NULL)
    int64_t max_leaf_rows = 0;         // largest owned leaf
    // E8 code hierarchy (E8 index): levels 1..e8_levels (e8hier.cu)
    int e8_levels = 0;
    std::vector<std::unique_ptr<blsh::DevBuf>> e8_key, e8_bu, e8_cum;
    std::vector<int32_t> e8_root_h;
    blsh::DevBuf e8_root;              // [G]
    blsh::DevBuf e8_ptrs;              // device pointer tables: keys, buckets, cum
    // kept build stages (keep_stages)
    blsh::DevBuf pt_leaf, pt_code, pt_key;
    bool has_pt = false;
    // query state
    mutable blsh::QueryWork qw;
    mutable blsh_stats stats{};
    mutable bool has_stages = false;
    mutable cudaEvent_t ev[10] = {};
};

namespace blsh {

// ---- build (rptree.cu, hash.cu, table.cu) --------------------------------------
// Host-side generator (params.cpp), reading R2.
void gen_params(uint64_t seed, int G, int M, int d, const float* Wleaf, float* A, float* b,
                float* dirs, double* jit);
// (a, b) of hash table `table` (table 0 = the ones gen_params draws).
void gen_table_params(uint64_t seed, int table, int G, int M, int d, const float* Wleaf, float* A, float* b);

// RP-tree over Xs [n][ds]; fills idx tree arrays; returns leaf segments of the
// final order (order_out [n] uint32 ids grouped by leaf, ascending id) and
// seg [G+1] (host).
void build_rptree(blsh_index& ix, const float* Xs, uint32_t* order_dev,
                  std::vector<int64_t>& seg, cudaStream_t s);

// Delta_A^2 of every leaf (R7 reductions over the members in ascending id), for
// the per-leaf W rule (R29).
void leaf_spread(const blsh_index& ix, const float* Xs, const uint32_t* order, const std::vector<int64_t>& seg,
                 std::vector<double>& da2_out, cudaStream_t s);

// Hash the points order[lo..hi) (grouped by leaf) with their leaf's params;
// writes sort entries; returns false when a code leaves the Morton range.
bool hash_points(const blsh_index& ix, const float* Xs, const uint32_t* order,
                 const std::vector<int64_t>& seg, int64_t pos_lo, int64_t pos_hi,
                 unsigned long long* key_hi, unsigned long long* key_lo, uint32_t* leaf,
                 uint32_t* id, int32_t* code_out /* nullable [n][M] by id */,
                 cudaStream_t s, const float* A = nullptr, const float* b = nullptr /* NULL: table 0's */);

// After sorting: buckets, offsets, permuted rows.
void build_table(blsh_index& ix, const float* Xs, const unsigned long long* key_hi,
                 const unsigned long long* key_lo, const uint32_t* leaf, const uint32_t* id,
                 int64_t n_owned, ScanTemp& scan, cudaStream_t s);

// The short-list screen's compact copy of the table: anchors, fp16 residual rows and
// per-row bound constants (resid.cu).  Call after build_table.
void build_screen_rows(blsh_index& ix, cudaStream_t s);
int screen_cols(int ds);

// Table l >= 1 (sorted entries of that table): bucket directory + pos via the
// inverse of table 0's permutation (inv0[id] = table-0 position).
void build_extra_table(const blsh_index& ix, ExtraTable& t, const unsigned long long* key_hi,
                       const unsigned long long* key_lo, const uint32_t* leaf, const uint32_t* id,
                       const uint32_t* inv0, int64_t n_owned, ScanTemp& scan, cudaStream_t s);
void invert_perm(const uint32_t* perm, int64_t n_owned, uint32_t* inv, cudaStream_t s);
// E8 index: the code hierarchy over the primary table's buckets (e8hier.cu).
void build_e8_hierarchy(blsh_index& ix, cudaStream_t s);

// ---- query (query.cu, shortlist.cu) ----------------------------------------------
void run_query(const blsh_index& ix, const float* Q, bool q_host, int64_t nq, int k,
               const blsh_query_params& p, int64_t* out_ids, float* out_d2,
               unsigned long long* out_packed, int64_t* out_ncand, bool out_host,
               int64_t* out_base);   // non-NULL: stop after a4 and write |A0(q)| (blsh_query_base_counts)
// blsh_query_pipelined: n_batches host batches, uploads/downloads overlapped with the search
void run_query_pipelined(const blsh_index& ix, int nb, const float* const* Q, int64_t nq, int k,
                         const blsh_query_params& p, int64_t* const* out_ids, float* const* out_d2,
                         int64_t* const* out_ncand);

void merge_lists(const unsigned long long* packed, int n_lists, int64_t nq, int k,
                 int64_t* out_ids, float* out_d2, cudaStream_t s);

}  // namespace blsh
