// shortlist_tiled.cu -- a5 with cross-query reuse (the default short-list).
//
// Queries are sorted by their bi-level code (leaf, home Morton key), so
// consecutive queries probe overlapping buckets.  A *tile* is QT = 32
// consecutive queries.  k_tile_prep turns the tile's candidate intervals into
// the sorted union of disjoint row segments, each with a 32-bit mask of the
// tile queries whose A(q) contains it (interval boundaries -> sort -> XOR
// toggles -> XOR prefix scan; a query's own intervals are disjoint).
// k_shortlist_tiled streams that union once: rows are staged into shared
// memory with 1-D TMA bulk copies (cp.async.bulk + mbarrier complete_tx,
// double-buffered, 16-byte padded row pitch so one-row-per-lane reads are
// bank-conflict free), and every warp scores the staged rows (one per lane)
// against its 4 tile queries held in shared memory (broadcast reads).  A row
// read from HBM once thus serves every query of the tile that needs it; the
// per-(row, query) arithmetic is the same fp32 direct form as k_shortlist
// (R22).  Each (work item, query) keeps a warp-register top-k; k_merge_tiled
// merges the items of a tile per query.
#include <algorithm>
#include <cstdio>
#include <cstdlib>
#include <cstring>

#include <cuda_fp16.h>

#include "internal.cuh"
#include "query_kernels.cuh"

namespace blsh {

namespace {

constexpr int QT = 32;            // queries per tile
constexpr int64_t kSmallBatch = 128;   // batches up to this size take the warp short-list
constexpr int kPrepThreads = 256;
constexpr int kRows = 32;         // rows per stage (one per lane)
constexpr int kTW = 8;            // warps per CTA (each owns 4 tile queries)

struct Seg {
    uint32_t start, len, mask, off;   // table rows [start, start+len), query mask, rows before it in the union
    uint32_t abase;                   // tile-local index of the anchor group of row `start` (screen K table)
    uint32_t atbase;                  // tile-local index of the 8-row atom of row `start` (fp16 screen rows)
};

// ---------------------------------------------------------------------------
// tile prep: union of the tile's candidate intervals, with query masks
// ---------------------------------------------------------------------------
__global__ void __launch_bounds__(kPrepThreads) k_tile_prep(const uint2* __restrict__ ivl, int T,
                                                            const uint32_t* __restrict__ qorder,
                                                            const int64_t* __restrict__ tile_off,
                                                            int segcap, Seg* __restrict__ segs,
                                                            int32_t* __restrict__ nseg,
                                                            int64_t* __restrict__ rows,
                                                            int64_t* __restrict__ nanch,
                                                            const uint32_t* __restrict__ rgrp,
                                                            int64_t* __restrict__ natom) {
    extern __shared__ uint32_t sm[];
    const int cap = 2 * QT * (T + 1);
    int npow = 1;
    while (npow < cap) npow <<= 1;
    uint32_t* bnd = sm;             // [npow] boundaries (sorted, then unique)
    uint32_t* tog = sm + npow;      // [npow] scratch -> toggles -> masks
    uint32_t* pos = tog + npow;     // [npow] unique positions
    __shared__ int s_cnt, s_nb;
    const int t = blockIdx.x;
    const int tid = threadIdx.x;
    if (tid == 0) s_cnt = 0;
    for (int i = tid; i < npow; i += kPrepThreads) bnd[i] = 0xFFFFFFFFu;
    __syncthreads();
    const int nint = QT * (T + 1);
    for (int i = tid; i < nint; i += kPrepThreads) {
        const int slot = i / (T + 1), p = i % (T + 1);
        const int64_t qp = tile_off[t] + slot;
        if (qp >= tile_off[t + 1]) continue;
        const uint2 iv = ivl[(size_t)qorder[qp] * (T + 1) + p];
        if (iv.y > iv.x) {
            const int at = atomicAdd(&s_cnt, 2);
            bnd[at] = iv.x;
            bnd[at + 1] = iv.y;
        }
    }
    __syncthreads();
    const int cnt = s_cnt;
    if (cnt == 0) {
        if (tid == 0) { nseg[t] = 0; rows[t] = 0; nanch[t] = 0; if (natom) natom[t] = 0; }
        return;
    }
    int np2 = 32;                                   // >= one warp of (padding) keys; npow >= 2 * QT
    while (np2 < cnt) np2 <<= 1;
    // bitonic sort of bnd[0..np2): steps with j >= 32 in shared memory, the
    // j <= 16 steps of each merge in registers (element i in lane i & 31, its
    // partner i ^ j one shuffle away), so a merge costs one barrier per
    // shared-memory step plus one for its register tail
    auto reg_steps = [&](int k2lo, int k2hi) {
        for (int i = tid; i < np2; i += kPrepThreads) {
            uint32_t v = bnd[i];
            for (int k2 = k2lo; k2 <= k2hi; k2 <<= 1) {
                const bool up = (i & k2) == 0;
                for (int j = min(k2 >> 1, 16); j > 0; j >>= 1) {
                    const uint32_t o = __shfl_xor_sync(BLSH_FULL, v, j);
                    v = (((i & j) == 0) == up) ? min(v, o) : max(v, o);
                }
            }
            bnd[i] = v;
        }
        __syncthreads();
    };
    reg_steps(2, 32);
    for (int k2 = 64; k2 <= np2; k2 <<= 1) {
        for (int j = k2 >> 1; j >= 32; j >>= 1) {
            for (int i = tid; i < np2; i += kPrepThreads) {
                const int ixj = i ^ j;
                if (ixj > i) {
                    const uint32_t a = bnd[i], b = bnd[ixj];
                    if ((a > b) == ((i & k2) == 0)) { bnd[i] = b; bnd[ixj] = a; }
                }
            }
            __syncthreads();
        }
        reg_steps(k2, k2);
    }
    // unique boundaries (exclusive scan of first-occurrence flags by warp 0)
    if (tid < 32) {
        const int per = (cnt + 31) / 32;
        const int lo = tid * per, hi = min(cnt, lo + per);
        uint32_t c = 0;
        for (int i = lo; i < hi; ++i) c += (i == 0 || bnd[i] != bnd[i - 1]) ? 1u : 0u;
        uint32_t inc = c;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const uint32_t y = __shfl_up_sync(BLSH_FULL, inc, o);
            if (tid >= o) inc += y;
        }
        uint32_t run = inc - c;
        for (int i = lo; i < hi; ++i) {
            pos[i] = run;
            run += (i == 0 || bnd[i] != bnd[i - 1]) ? 1u : 0u;
        }
        if (tid == 31) s_nb = (int)inc;
    }
    __syncthreads();
    const int nb = s_nb;
    for (int i = tid; i < cnt; i += kPrepThreads)
        if (i == 0 || bnd[i] != bnd[i - 1]) tog[pos[i]] = bnd[i];
    __syncthreads();
    for (int i = tid; i < nb; i += kPrepThreads) bnd[i] = tog[i];
    __syncthreads();
    for (int i = tid; i < npow; i += kPrepThreads) tog[i] = 0u;
    __syncthreads();
    for (int i = tid; i < nint; i += kPrepThreads) {     // XOR toggles at both ends of every interval
        const int slot = i / (T + 1), p = i % (T + 1);
        const int64_t qp = tile_off[t] + slot;
        if (qp >= tile_off[t + 1]) continue;
        const uint2 iv = ivl[(size_t)qorder[qp] * (T + 1) + p];
        if (iv.y > iv.x) {
            int lo = 0, hi = nb;
            while (lo < hi) { const int m = (lo + hi) >> 1; if (bnd[m] < iv.x) lo = m + 1; else hi = m; }
            const int is = lo;
            hi = nb;
            while (lo < hi) { const int m = (lo + hi) >> 1; if (bnd[m] < iv.y) lo = m + 1; else hi = m; }
            atomicXor(&tog[is], 1u << slot);
            atomicXor(&tog[lo], 1u << slot);
        }
    }
    __syncthreads();
    if (tid < 32) {                                        // inclusive XOR scan -> mask of [bnd[i], bnd[i+1])
        const int per = (nb + 31) / 32;
        const int lo = tid * per, hi = min(nb, lo + per);
        uint32_t x = 0;
        for (int i = lo; i < hi; ++i) x ^= tog[i];
        uint32_t inc = x;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const uint32_t y = __shfl_up_sync(BLSH_FULL, inc, o);
            if (tid >= o) inc ^= y;
        }
        uint32_t run = inc ^ x;
        for (int i = lo; i < hi; ++i) { run ^= tog[i]; tog[i] = run; }
    }
    __syncthreads();
    if (tid < 32) {                                        // emit segments with a non-empty mask, in order
        int out = 0;
        uint32_t off = 0;
        Seg* S = segs + (size_t)t * segcap;
        for (int base = 0; base < nb - 1; base += 32) {
            const int i = base + tid;
            const bool v = i < nb - 1 && tog[i] != 0u;
            const unsigned bm = __ballot_sync(BLSH_FULL, v);
            const uint32_t len = v ? bnd[i + 1] - bnd[i] : 0u;
            uint32_t inc = len;
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                const uint32_t y = __shfl_up_sync(BLSH_FULL, inc, o);
                if (tid >= o) inc += y;
            }
            if (v) S[out + __popc(bm & lanemask_lt())] = Seg{bnd[i], len, tog[i], off + inc - len, 0u, 0u};
            off += __shfl_sync(BLSH_FULL, inc, 31);
            out += __popc(bm);
        }
        __syncwarp();
        // Runs of table rows the union touches, numbered in row order: anchor groups
        // (resid.cu) and 8-row atoms.  Segment i covers runs [a0, a1]; it shares a0 with
        // segment i-1 when that one ends in it.  Returns the number of distinct runs.
        auto number_runs = [&](auto run_of, bool anchors) {
            uint32_t na = 0, prev_last = 0xFFFFFFFFu;
            for (int base = 0; base < out; base += 32) {
                const int i = base + tid;
                uint32_t a0 = 0, a1 = 0;
                if (i < out) {
                    const Seg sg = S[i];
                    a0 = run_of(sg.start);
                    a1 = run_of(sg.start + sg.len - 1);
                }
                const uint32_t up = __shfl_up_sync(BLSH_FULL, a1, 1);
                const uint32_t pl = tid == 0 ? prev_last : up;
                const uint32_t shared = (i < out && pl == a0) ? 1u : 0u;
                const uint32_t c = i < out ? a1 - a0 + 1u - shared : 0u;
                uint32_t inc = c;
#pragma unroll
                for (int o = 1; o < 32; o <<= 1) {
                    const uint32_t y = __shfl_up_sync(BLSH_FULL, inc, o);
                    if (tid >= o) inc += y;
                }
                if (i < out) {
                    if (anchors) S[i].abase = na + inc - c - shared;
                    else S[i].atbase = na + inc - c - shared;
                }
                na += __shfl_sync(BLSH_FULL, inc, 31);
                prev_last = __shfl_sync(BLSH_FULL, a1, min(31, out - 1 - base));
            }
            return na;
        };
        const uint32_t na = number_runs([&](uint32_t r) { return rgrp ? rgrp[r] : 0u; }, true);
        const uint32_t nat = number_runs([](uint32_t r) { return r >> 3; }, false);
        if (tid == 0) { nseg[t] = out; rows[t] = off; nanch[t] = na; if (natom) natom[t] = 8 * (int64_t)nat; }
    }
}

// Expand the tiles' segment lists to one (table row, query mask) entry per union row,
// at rows_off[tile] + (row index within the tile's union): the TC short-list reads its
// block metadata with one coalesced load instead of walking the segment list.
// Each entry also carries the row's K-table slot (aoff[tile] + the tile-local index of
// its anchor block); the first row of every (segment, anchor block) records the slot's
// anchor block (a block shared by two segments is written twice with the same value).
__global__ void __launch_bounds__(256) k_expand_rows(const Seg* __restrict__ segs, const int32_t* __restrict__ nseg,
                                                     int segcap, const int64_t* __restrict__ rows_off,
                                                     const int64_t* __restrict__ aoff, uint4* __restrict__ rowinfo,
                                                     uint32_t* __restrict__ slot_anchor,
                                                     const uint32_t* __restrict__ rgrp) {
    const int64_t t = blockIdx.x;
    const Seg* S = segs + (size_t)t * segcap;
    uint4* out = rowinfo + rows_off[t];
    const int64_t ab = aoff[t];
    const int ns = nseg[t];
    const int lane = threadIdx.x & 31;
    for (int sI = threadIdx.x >> 5; sI < ns; sI += 8) {
        const Seg sg = S[sI];
        const uint32_t a0 = rgrp ? rgrp[sg.start] : 0u;
        for (uint32_t i = lane; i < sg.len; i += 32) {
            const uint32_t row = sg.start + i;
            const uint32_t grp = rgrp ? rgrp[row] : 0u;
            const int64_t slot = ab + sg.abase + (grp - a0);
            out[sg.off + i] = make_uint4(row, sg.mask, (uint32_t)slot, 0u);
            if (slot_anchor && (i == 0 || rgrp[row - 1] != grp)) slot_anchor[slot] = grp;
        }
    }
}

// Work items of a tile: consecutive row ranges of <= chr union rows; with the fp16 screen
// (rowinfo != NULL) an item also spans < amax anchor blocks (its anchor columns of the
// MMA, k_screen_f16).  One thread per tile walks its rows; the anchor slot (rowinfo.z) is
// non-decreasing along a tile's rows.  Pass 1 (item_r0 == NULL) counts, pass 2 writes
// every item's first row (item_r0[item_off[t] + i], tile-relative).
// fp16 screen: the tile's union at 8-row-atom granularity, one entry per atom row
// (atom-row index = 8 x the atom's tile-local index + (row & 7)): union rows carry (table row,
// query mask, K slot); the other rows of a touched atom carry mask 0 and the K slot of the
// atom's previous union row (or its first), so the slot stays non-decreasing along the
// tile's rows (k_tile_items splits items on it).  One CTA per tile, one thread per atom: the
// thread finds the first segment touching its atom (binary search over the segments' last
// atoms, which are non-decreasing), walks the atom's 8 rows through that segment and the
// later ones starting inside the atom, fills the non-union rows' K slots in registers; the
// CTA's 256 atoms (32 KB) leave through shared memory (XOR-swizzled 16-byte slots) as
// coalesced stores.  Every entry is written once.
__global__ void __launch_bounds__(256) k_expand_atoms(const Seg* __restrict__ segs, const int32_t* __restrict__ nseg,
                                                      int segcap, const int64_t* __restrict__ arows_off,
                                                      const int64_t* __restrict__ aoff, const uint32_t* __restrict__ rgrp,
                                                      uint4* __restrict__ rowinfo, uint32_t* __restrict__ slot_anchor) {
    __shared__ uint4 stage[256 * 8];
    const int64_t t = blockIdx.x;
    const Seg* S = segs + (size_t)t * segcap;
    uint4* out = rowinfo + arows_off[t];
    const int64_t ab = aoff[t];
    const int ns = nseg[t];
    const int64_t nat = (arows_off[t + 1] - arows_off[t]) >> 3;
    const int tid = threadIdx.x;
    auto last_atom = [&](const Seg& g) { return (int64_t)g.atbase + ((g.start + g.len - 1) >> 3) - (g.start >> 3); };
    int lo = 0;
    for (int64_t base = 0; base < nat; base += 256) {
        const int64_t A = base + tid;
        if (A < nat) {
            int l = lo, h = ns - 1;
            while (l < h) {
                const int m = (l + h) >> 1;
                if (last_atom(S[m]) >= A) h = m;
                else l = m + 1;
            }
            lo = l;
            int sj = l;
            Seg cs = S[sj];
            const uint32_t at = (cs.start >> 3) + (uint32_t)(A - cs.atbase);
            uint32_t cg0 = rgrp[cs.start];
            uint4 e[8];
#pragma unroll
            for (int r = 0; r < 8; ++r) {
                const uint32_t row = at * 8u + (uint32_t)r;
                while (row >= cs.start + cs.len && sj + 1 < ns && S[sj + 1].start <= row) {
                    cs = S[++sj];
                    cg0 = rgrp[cs.start];
                }
                if (row >= cs.start && row < cs.start + cs.len) {
                    const uint32_t grp = rgrp[row];
                    const int64_t slot = ab + cs.abase + (grp - cg0);
                    e[r] = make_uint4(row, cs.mask, (uint32_t)slot, 0u);
                    if (row == cs.start || rgrp[row - 1] != grp) slot_anchor[slot] = grp;
                } else {
                    e[r] = make_uint4(row, 0u, 0u, 0u);
                }
            }
            uint32_t cur = 0;
            bool found = false;
#pragma unroll
            for (int r = 0; r < 8; ++r)
                if (!found && e[r].y != 0u) { cur = e[r].z; found = true; }
#pragma unroll
            for (int r = 0; r < 8; ++r) {
                if (e[r].y != 0u) cur = e[r].z;
                else e[r].z = cur;
                stage[tid * 8 + (r ^ (tid & 7))] = e[r];
            }
        }
        __syncthreads();
        const int cnt = (int)min((int64_t)256, nat - base) * 8;
        uint4* o = out + base * 8;
        for (int i = tid; i < cnt; i += 256) {
            const int a8 = i >> 3, r = i & 7;
            o[i] = stage[a8 * 8 + (r ^ (a8 & 7))];
        }
        __syncthreads();
    }
}

__global__ void k_tile_items(const int64_t* __restrict__ rows, const int64_t* __restrict__ rows_off,
                             const uint4* __restrict__ rowinfo, int64_t ntiles, int chr, int amax,
                             int64_t* __restrict__ items, const int64_t* __restrict__ item_off,
                             int64_t* __restrict__ item_r0) {
    const int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (t >= ntiles) return;
    const int64_t R = rows[t];
    const uint4* RI = rowinfo ? rowinfo + rows_off[t] : nullptr;
    int64_t r = 0, it = 0;
    while (r < R) {
        int64_t e = min(r + (int64_t)chr, R);
        if (RI) {
            const uint32_t lim = RI[r].z + (uint32_t)amax;   // first slot that no longer fits
            if (RI[e - 1].z >= lim) {
                int64_t lo = r + 1, hi = e - 1;                // smallest row with slot >= lim
                while (lo < hi) {
                    const int64_t m = (lo + hi) >> 1;
                    if (RI[m].z >= lim) hi = m;
                    else lo = m + 1;
                }
                e = lo & ~(int64_t)7;              // whole atoms (an atom spans <= 8 groups)
                if (e <= r) e = r + 8;
            }
        }
        if (item_r0) item_r0[item_off[t] + it] = r;
        ++it;
        r = e;
    }
    if (!item_r0) items[t] = it;
}

// ---------------------------------------------------------------------------
// TMA bulk copy + mbarrier
// ---------------------------------------------------------------------------
__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t* bar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes) : "memory");
}
// Warp-wide wait (every caller is a whole warp).  Lanes may leave the try_wait
// loop on different iterations; the __syncwarp reconverges them so that the
// warp collectives that follow take the converged fast path.
#ifndef BLSH_SPIN_WAIT
#define BLSH_SPIN_WAIT 0
#endif
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
#if BLSH_SPIN_WAIT
    asm volatile(
        "{\n\t.reg .pred p;\n"
        "WAIT_%=:\n\t"
        "mbarrier.test_wait.parity.shared::cta.b64 p, [%0], %1;\n\t"
        "@!p bra WAIT_%=;\n\t}" ::"r"(smem_u32(bar)),
        "r"(parity)
        : "memory");
#else
    asm volatile(
        "{\n\t.reg .pred p;\n"
        "WAIT_%=:\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t"
        "@!p bra WAIT_%=;\n\t}" ::"r"(smem_u32(bar)),
        "r"(parity)
        : "memory");
#endif
    __syncwarp();
}
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                 ::"r"(smem_u32(dst)), "l"(src), "r"(bytes), "r"(smem_u32(bar))
                 : "memory");
}

struct TiledArgs {
    int64_t nq, ntiles, n_items;
    int d, ds, k, chr, segcap;
    const float* Q;
    const float* Xp;
    const uint32_t* perm;
    const uint32_t* qorder;
    const Seg* segs;
    const int32_t* nseg;
    const int64_t* rows;       // [ntiles] union rows per tile
    const int64_t* item_off;   // [ntiles+1]
    const int64_t* item_r0;    // [n_items] first union row of each item (tile-relative); the item ends at
                               // the next item's first row (or the tile's last row)
    unsigned long long* partials;   // [n_items][QT][k]
    const int64_t* tile_off;        // [ntiles+1] sorted-query positions of each tile
    const int32_t* tile_of;         // [nq] tile of each sorted position
    unsigned long long* counters;   // [0] (row, query) pairs evaluated, [1] screen survivors (TC)
    float* dbg;                     // optional (BLSH_TC_DEBUG): item 0, block 0 dots / |x'|^2 / rows
    unsigned long long* sbuf;       // TC: [n_items][QT][scap] buffered (lower bound, row) pairs
    int scap;
    int scapw;                      // per list (scap = nlist x scapw)
    int nlist;                      // TC screens: buffered-pair lists per (item, query): epilogue warps
    int dbgmode;                    // ablation (BLSH_TC_MODE): 1 skip screen, 2 skip row loads, 4 skip MMA, 32 phase timers
    unsigned long long* tstamp;     // BLSH_TC_MODE & 32: [n_items][8] globaltimer stamps per phase
    const int64_t* rows_off;        // [ntiles + 1] union rows before each tile
    const uint4* rowinfo;           // TC: [total rows] (table row, query mask, K slot, 0) per union row
    int dr;                         // screen: fp16 columns of the compact rows
    const __half* Rh;               // screen: fp16 rows, panel-major swizzled 8-row atoms (resid.cu)
    int64_t natom;                  // screen: atoms of the table (Rh panel stride = natom KB)
    const float4* rconst;           // screen: [n] per-row bound constants
    const float* ktab;              // screen: [K slots][QT] K_aj = |q_j - a|^2
    const float* anc;               // screen: [anchor groups][dr] fp32 anchors
    const uint32_t* slot_anchor;    // screen: [K slots] anchor group of each slot
    uint32_t* ufin;                 // TC -> k_tc_rescore: [n_items][QT] final screen bound U_j (fp32 bits)
    int32_t* scnt;                  // TC -> k_tc_rescore: [n_items][QT][4] buffered pairs per epilogue warp
};

// Tile of a work item (binary search over item_off) and the item's union rows [r0, r1).
__device__ __forceinline__ int64_t item_tile_rows(const TiledArgs& a, int64_t item, int64_t* r0, int64_t* r1) {
    int64_t lo = 0, hi = a.ntiles;
    while (hi - lo > 1) {
        const int64_t mid = (lo + hi) >> 1;
        if (a.item_off[mid] <= item) lo = mid;
        else hi = mid;
    }
    *r0 = a.item_r0[item];
    *r1 = item + 1 < a.item_off[lo + 1] ? a.item_r0[item + 1] : a.rows[lo];
    return lo;
}

struct TopK {
    unsigned long long e0, e1;
};

__device__ __forceinline__ unsigned long long topk_thr(const TopK& t, int k) {
    return __shfl_sync(BLSH_FULL, k <= 32 ? t.e0 : t.e1, (k - 1) & 31);
}

__device__ __forceinline__ void topk_insert(TopK& t, unsigned long long v, int lane) {
    const int pos = __popc(__ballot_sync(BLSH_FULL, t.e0 < v)) + __popc(__ballot_sync(BLSH_FULL, t.e1 < v));
    const unsigned long long up0 = __shfl_up_sync(BLSH_FULL, t.e0, 1);
    unsigned long long up1 = __shfl_up_sync(BLSH_FULL, t.e1, 1);
    const unsigned long long last0 = __shfl_sync(BLSH_FULL, t.e0, 31);
    if (lane == 0) up1 = last0;
    const int i1 = lane + 32;
    t.e1 = i1 > pos ? up1 : (i1 == pos ? v : t.e1);
    t.e0 = lane > pos ? up0 : (lane == pos ? v : t.e0);
}

// Offer one key per lane (kEmpty = none) to a warp top-k.
__device__ __forceinline__ void topk_offer(TopK& tk, unsigned long long& thr, unsigned long long key, int k, int lane) {
    unsigned m = __ballot_sync(BLSH_FULL, key < thr);
    while (m) {
        const int src = __ffs(m) - 1;
        m &= m - 1;
        const unsigned long long v = __shfl_sync(BLSH_FULL, key, src);
        if (v < thr) {
            topk_insert(tk, v, lane);
            thr = topk_thr(tk, k);
        }
    }
}


#include "tiled_kernel.cuh"
#include "tc_kernel.cuh"
#include "screen_kernel.cuh"

__global__ void __launch_bounds__(256) k_merge_tiled(TiledArgs a, const int32_t* __restrict__ qoor,
                                                     const int64_t* __restrict__ cnt, int64_t* out_ids, float* out_d2,
                                                     unsigned long long* out_packed, int64_t* out_ncand) {
    const int lane = threadIdx.x & 31;
    const int64_t pos = blockIdx.x * (int64_t)(blockDim.x >> 5) + (threadIdx.x >> 5);
    if (pos >= a.nq) return;
    const int64_t q = a.qorder[pos];
    const int64_t tile = a.tile_of[pos];
    const int slot = (int)(pos - a.tile_off[tile]);
    const int k = a.k;
    TopK tk{kEmpty, kEmpty};
    unsigned long long thr = kEmpty;
    for (int64_t it = a.item_off[tile]; it < a.item_off[tile + 1]; ++it) {
        const unsigned long long* L = a.partials + ((size_t)it * QT + slot) * k;
        const unsigned long long l0 = lane < k ? L[lane] : kEmpty;
        const unsigned long long l1 = lane + 32 < k ? L[lane + 32] : kEmpty;
        for (int j = 0; j < k; ++j) {
            const unsigned long long v = __shfl_sync(BLSH_FULL, j < 32 ? l0 : l1, j & 31);
            if (v >= thr) break;
            topk_insert(tk, v, lane);
            thr = topk_thr(tk, k);
        }
    }
#pragma unroll
    for (int h = 0; h < 2; ++h) {
        const int i = lane + 32 * h;
        if (i >= k) continue;
        const unsigned long long e = h ? tk.e1 : tk.e0;
        if (out_packed) out_packed[(size_t)q * k + i] = e == kEmpty ? kPadPacked : e;
        if (out_ids) out_ids[(size_t)q * k + i] = e == kEmpty ? -1 : (int64_t)(uint32_t)(e & 0xFFFFFFFFull);
        if (out_d2) out_d2[(size_t)q * k + i] = e == kEmpty ? __int_as_float(0x7F800000) : __uint_as_float((uint32_t)(e >> 32));
    }
    if (lane == 0 && out_ncand) out_ncand[q] = (qoor[q] & 2) ? 0 : cnt[q];
}

__global__ void k_qsort_keys(const Key128* __restrict__ qkey, const int32_t* __restrict__ qleaf,
                             const int32_t* __restrict__ qoor, int64_t nq, unsigned long long* __restrict__ hi,
                             unsigned long long* __restrict__ lo, uint32_t* __restrict__ leaf, uint32_t* __restrict__ id) {
    const int64_t q = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (q >= nq) return;
    // Sorting only groups similar queries into tiles (results do not depend on the order):
    // the low 64 key bits are the Morton interleave of the low bit-planes of the codes
    // (R9), which is where the queries of one leaf differ; the high bit-planes are mostly
    // the offset-binary sign pattern.  hi = 0 is a constant digit the radix sort skips.
    const Key128 k = qkey[q];
    hi[q] = 0ull;
    lo[q] = k.lo;
    leaf[q] = (qoor[q] & 6) ? 0xFFFFu : (uint32_t)qleaf[q];   // not owned / non-finite (R30): own tiles
    id[q] = (uint32_t)q;
}

// ---------------------------------------------------------------------------
// tile formation: consecutive sorted queries, at most QT per tile, a new tile
// at every leaf change and wherever two consecutive queries are far apart
// (> 16 x the median consecutive squared distance), so a tile's queries sit
// in one region of space (the TC screen's error bound grows with |q - c|).
// ---------------------------------------------------------------------------
__global__ void k_consec_d2(const float* __restrict__ Q, int ds, const uint32_t* __restrict__ qorder, int64_t nq,
                            int64_t* __restrict__ d2bits) {
    const int lane = threadIdx.x & 31;
    const int64_t i = blockIdx.x * (int64_t)(blockDim.x >> 5) + (threadIdx.x >> 5) + 1;
    if (i >= nq) return;
    const float4* a = reinterpret_cast<const float4*>(Q + (size_t)qorder[i] * ds);
    const float4* b = reinterpret_cast<const float4*>(Q + (size_t)qorder[i - 1] * ds);
    float s = 0.f;
    for (int v = lane; v < (ds >> 2); v += 32) {
        const float4 x = a[v], y = b[v];
        const float dx = x.x - y.x, dy = x.y - y.y, dz = x.z - y.z, dw = x.w - y.w;
        s += dx * dx + dy * dy + dz * dz + dw * dw;
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(BLSH_FULL, s, o);
    if (lane == 0) d2bits[i - 1] = (int64_t)__float_as_uint(s);
}

__global__ void k_tile_flags(const int64_t* __restrict__ d2bits, const int64_t* __restrict__ med,
                             const int32_t* __restrict__ qleaf, const int32_t* __restrict__ qoor,
                             const uint32_t* __restrict__ qorder, int64_t nq, uint8_t* __restrict__ brk,
                             float jump) {
    const int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (i >= nq) return;
    if (i == 0) { brk[0] = 1; return; }
    const uint32_t a = qorder[i], b = qorder[i - 1];
    const uint32_t la = (qoor[a] & 6) ? 0xFFFFu : (uint32_t)qleaf[a];
    const uint32_t lb = (qoor[b] & 6) ? 0xFFFFu : (uint32_t)qleaf[b];
    const float lim = jump * __uint_as_float((uint32_t)*med);
    brk[i] = (la != lb || __uint_as_float((uint32_t)d2bits[i - 1]) > lim) ? 1 : 0;
}

__global__ void k_run_start(const uint8_t* __restrict__ brk, const int64_t* __restrict__ excl, int64_t nq,
                            int64_t* __restrict__ run_start) {
    const int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (i < nq && brk[i]) run_start[excl[i]] = i;
}

__global__ void k_tile_start(const uint8_t* __restrict__ brk, const int64_t* __restrict__ excl,
                             const int64_t* __restrict__ run_start, int64_t nq, uint8_t* __restrict__ ts) {
    const int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (i >= nq) return;
    const int64_t rid = excl[i] + brk[i] - 1;
    ts[i] = ((i - run_start[rid]) % QT == 0) ? 1 : 0;
}

__global__ void k_tile_scatter(const uint8_t* __restrict__ ts, const int64_t* __restrict__ excl, int64_t nq,
                               int64_t* __restrict__ tile_off, int32_t* __restrict__ tile_of) {
    const int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (i >= nq) return;
    const int64_t t = excl[i] + ts[i] - 1;
    tile_of[i] = (int32_t)t;
    if (ts[i]) tile_off[t] = i;
    if (i == nq - 1) tile_off[t + 1] = nq;
}

}  // namespace

size_t tiled_smem_bytes(int ds) { return 1024 + (size_t)QT * ds * 4 + (size_t)kStages * 32 * (ds + 4) * 4; }

size_t tc_smem_bytes(int ds) {
    return ((sizeof(TcSmem) + 1023) & ~size_t(1023)) + (size_t)QT * ds * 4 + (size_t)kTcSlots * kTcChunkBytes;
}

// BLSH_SCREEN=tf32: the round-1 TF32 screen (k_shortlist_tc, converter warps) instead of
// the fp16 compact-table screen (k_screen_f16); read once per process.
static int screen_variant() {
    static const int v = [] {
        const char* e = std::getenv("BLSH_SCREEN");
        return (e && std::strcmp(e, "tf32") == 0) ? 1 : 0;
    }();
    return v;
}

int64_t small_batch_limit() { return kSmallBatch; }

int shortlist_kind(int64_t nq, int ds, int dr, int T, int k) {
    const char* mode = std::getenv("BLSH_SHORTLIST");
    if (mode && std::strcmp(mode, "warp") == 0) return 0;
    // small batches (<= 4 tiles): the tiled path's planning launches and host round trips
    // (~0.6 ms) exceed the warp short-list's whole run (profiles/r02/c5_sweep.jsonl, B <= 100)
    // batches of up to 1 024 queries with few probes also stream faster without tiles: C5 at
    // 1 000 queries, T = 16 multiprobe / T = 8 E8: warp 0.94 / 0.98 ms vs tiled 1.17 / 1.20 ms;
    // with T = 64 Morton-curve probes the tiles win (1.38 vs 1.58 ms) (profiles/r02/c5_sweep_final)
    if (!mode && (nq <= kSmallBatch || (nq <= 1024 && nq * (int64_t)T <= 16384))) return 0;
    // large k (64 < k <= 512): the fp16 screen (kk lists) + exact keys per query + k_select;
    // beyond, or without the fp16 screen: the warp short-list emitting every key + k_select
    if (k > 64 && (k > kSxMaxKLarge || screen_variant() != 0 || (mode && std::strcmp(mode, "simt") == 0))) return 0;
    int cap = 2 * QT * (T + 1), npow = 1;
    while (npow < cap) npow <<= 1;
    if ((size_t)3 * npow * 4 > 227 * 1024) return 0;   // tile prep does not fit
    const bool simt_ok = k <= 64 && tiled_smem_bytes(ds) <= 227 * 1024;
    const bool tc_ok = screen_variant() == 1
                           ? (k <= kTcMaxK && ds % kTcChunk == 0 && ds <= 512 && tc_smem_bytes(ds) <= 227 * 1024)
                           : ((k <= kSxMaxK || k <= kSxMaxKLarge) && dr >= 64 && dr <= kSxMaxDr && screen_stages(dr) > 0);
    if (mode && std::strcmp(mode, "simt") == 0) return simt_ok ? 1 : 0;
    if (tc_ok) return 2;
    return simt_ok ? 1 : 0;
}

// Sort the active queries by (leaf, home key): qorder[pos] = query.
void sort_queries(const QueryArgs& a, SortBufs& sb, uint32_t* qorder, cudaStream_t s, int* launches) {
    const int64_t nq = a.nq;
    for (int i = 0; i < 2; ++i) {
        sb.hi[i].ensure((size_t)nq * 8);
        sb.lo[i].ensure((size_t)nq * 8);
        sb.leaf[i].ensure((size_t)nq * 4);
        sb.id[i].ensure((size_t)nq * 4);
    }
    k_qsort_keys<<<(unsigned)((nq + 255) / 256), 256, 0, s>>>(a.qkey, a.qleaf, a.qoor, nq,
                                                               sb.hi[0].as<unsigned long long>(),
                                                               sb.lo[0].as<unsigned long long>(),
                                                               sb.leaf[0].as<uint32_t>(), sb.id[0].as<uint32_t>());
    BLSH_LAUNCH_CHECK();
    ++*launches;
    int passes = 0;
    const int cur = radix_sort_entries(sb, nq, s, &passes);
    *launches += (nq > 1 ? 1 : 0) + passes * 5;
    BLSH_CUDA(cudaMemcpyAsync(qorder, sb.id[cur].p, (size_t)nq * 4, cudaMemcpyDeviceToDevice, s));
}

// Query tiles (DESIGN §7 "Tiling"): consecutive sorted queries cut at leaf changes and
// large jumps.  Needs only a1/a2 outputs, so run_query issues it on a side stream while
// a3/a4 run; returns the tile count (host-synchronised on `s`).
int64_t plan_tiles(const QueryArgs& a, const uint32_t* qorder, DevBuf& tilebuf, ScanTemp& scan, cudaStream_t s,
                   int* launches) {
    const int64_t nq = a.nq;
    // tile arrays are sized for the worst case (one query per tile)
    const size_t slot = (((size_t)(nq + 1) * 8) + 255) & ~size_t(255);
    tilebuf.ensure(slot * 16 + 256);
    char* tb = tilebuf.as<char>();
    unsigned long long* counters = reinterpret_cast<unsigned long long*>(tb + 5 * slot);
    BLSH_CUDA(cudaMemsetAsync(counters, 0, 64, s));
    int64_t* tile_off = reinterpret_cast<int64_t*>(tb + 6 * slot);
    int32_t* tile_of = reinterpret_cast<int32_t*>(tb + 7 * slot);
    int64_t* d2bits = reinterpret_cast<int64_t*>(tb + 8 * slot);
    int64_t* fexcl = reinterpret_cast<int64_t*>(tb + 9 * slot);
    int64_t* run_start = reinterpret_cast<int64_t*>(tb + 10 * slot);
    uint8_t* brk = reinterpret_cast<uint8_t*>(tb + 11 * slot);
    uint8_t* tst = reinterpret_cast<uint8_t*>(tb + 11 * slot + (slot >> 1));
    int64_t* med = reinterpret_cast<int64_t*>(tb + 12 * slot);
    {
        const unsigned g256 = (unsigned)((nq + 255) / 256);
        BLSH_CUDA(cudaMemsetAsync(med, 0, 8, s));
        if (nq > 1) {
            k_consec_d2<<<(unsigned)((nq + 7) / 8), 256, 0, s>>>(a.Q, a.ds, qorder, nq, d2bits);
            BLSH_LAUNCH_CHECK();
            launch_median(d2bits, nq - 1, med, s);
            *launches += 2;
        }
        // cut a tile where consecutive queries are > 2048x the median squared step apart: at 4-512x
        // c3's tiles (Zipf clusters, 5% between-cluster queries) were fragmented -- 99 M union rows,
        // screen 16.1 ms; 2048x: 47 M, 9.0 ms (512 k -> 819 k q/s) with c4 unchanged; at 8192x the
        // tiles span clusters, the screen's bound loosens and c4 and c3 slow down (r02ax sweep)
        float jump = 2048.0f;
        if (const char* e = std::getenv("BLSH_TILE_JUMP")) jump = (float)std::atof(e);   // (experiments)
        k_tile_flags<<<g256, 256, 0, s>>>(d2bits, med, a.qleaf, a.qoor, qorder, nq, brk, jump);
        BLSH_LAUNCH_CHECK();
        scan_exclusive_u8(brk, fexcl, nq, scan, s);
        k_run_start<<<g256, 256, 0, s>>>(brk, fexcl, nq, run_start);
        BLSH_LAUNCH_CHECK();
        k_tile_start<<<g256, 256, 0, s>>>(brk, fexcl, run_start, nq, tst);
        BLSH_LAUNCH_CHECK();
        scan_exclusive_u8(tst, fexcl, nq, scan, s);
        k_tile_scatter<<<g256, 256, 0, s>>>(tst, fexcl, nq, tile_off, tile_of);
        BLSH_LAUNCH_CHECK();
        *launches += 10;
    }
    int64_t ntiles = 0;
    BLSH_CUDA(cudaMemcpyAsync(&ntiles, fexcl + nq, 8, cudaMemcpyDeviceToHost, s));
    BLSH_CUDA(cudaStreamSynchronize(s));
    return ntiles;
}

void run_tiled_shortlist(const QueryArgs& a, const uint32_t* qorder, int k, DevBuf& segbuf, DevBuf& tilebuf,
                         DevBuf& rowbuf,
                         DevBuf& partials, DevBuf& keybuf, ScanTemp& scan, int64_t* out_ids, float* out_d2,
                         unsigned long long* out_packed, int64_t* out_ncand, const float* Xp, const uint32_t* perm,
                         cudaStream_t s, int* launches, int64_t* n_items_out, int* chr_out, int64_t* rows_out,
                         cudaEvent_t ev_sl0, cudaEvent_t ev_mid, cudaEvent_t ev_sl1, int64_t* pairs_out,
                         int64_t* kept_out, double* qload_rows_out, int kind, int64_t ntiles,
                         int64_t* kslots_out, int* screen_kind_out) {
    const int64_t nq = a.nq;
    const int T = a.T;
    const int segcap = 2 * QT * (T + 1);
    const size_t slot = (((size_t)(nq + 1) * 8) + 255) & ~size_t(255);
    char* tb = tilebuf.as<char>();
    unsigned long long* counters = reinterpret_cast<unsigned long long*>(tb + 5 * slot);
    int64_t* tile_off = reinterpret_cast<int64_t*>(tb + 6 * slot);
    int32_t* tile_of = reinterpret_cast<int32_t*>(tb + 7 * slot);
    segbuf.ensure((size_t)std::max<int64_t>(ntiles, 1) * segcap * sizeof(Seg));
    int32_t* nseg = reinterpret_cast<int32_t*>(tb);
    int64_t* rows = reinterpret_cast<int64_t*>(tb + slot);
    int64_t* rows_off = reinterpret_cast<int64_t*>(tb + 2 * slot);
    int64_t* items = reinterpret_cast<int64_t*>(tb + 3 * slot);
    int64_t* item_off = reinterpret_cast<int64_t*>(tb + 4 * slot);
    int npow = 1;
    while (npow < segcap) npow <<= 1;
    const size_t prep_smem = (size_t)3 * npow * 4;
    int64_t* nanch = reinterpret_cast<int64_t*>(tb + 13 * slot);   // anchor groups per tile (screen K table)
    int64_t* aoff = reinterpret_cast<int64_t*>(tb + 14 * slot);
    int64_t* arows = reinterpret_cast<int64_t*>(tb + 15 * slot);   // fp16 screen: atom rows per tile
    const bool use_tc = kind == 2;   // chosen by shortlist_kind()
    const bool use_f16 = use_tc && screen_variant() == 0;
    BLSH_CUDA(cudaFuncSetAttribute(k_tile_prep, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)prep_smem));
    k_tile_prep<<<(unsigned)ntiles, kPrepThreads, prep_smem, s>>>(a.ivl, T, qorder, tile_off, segcap,
                                                                  segbuf.as<Seg>(), nseg, rows, nanch, a.rgrp,
                                                                  use_f16 ? arows : nullptr);
    BLSH_LAUNCH_CHECK();
    ++*launches;
    // the rows the short-list kernels walk: union rows, or (fp16 screen) the rows of the union's atoms
    int64_t* wrows = use_f16 ? arows : rows;
    scan_exclusive_i64(wrows, rows_off, ntiles, scan, s);
    *launches += 3;
    if (use_f16) {
        scan_exclusive_i64(nanch, aoff, ntiles, scan, s);
        *launches += 3;
    }
    int64_t tot2[2] = {0, 0};   // walked rows, K slots
    BLSH_CUDA(cudaMemcpyAsync(&tot2[0], rows_off + ntiles, 8, cudaMemcpyDeviceToHost, s));
    if (use_f16) BLSH_CUDA(cudaMemcpyAsync(&tot2[1], aoff + ntiles, 8, cudaMemcpyDeviceToHost, s));
    BLSH_CUDA(cudaStreamSynchronize(s));
    const int64_t total_rows = tot2[0], total_slots = tot2[1];
    // per-union-row entries (TC paths), the fp16 screen's K table and anchor list, item first rows
    const size_t rinfo_bytes = ((size_t)std::max<int64_t>(total_rows, 1) * 16 + 255) & ~size_t(255);
    const size_t ktab_bytes = ((size_t)std::max<int64_t>(total_slots, 1) * QT * 4 + 255) & ~size_t(255);
    const size_t slot_bytes = ((size_t)std::max<int64_t>(total_slots, 1) * 4 + 255) & ~size_t(255);
    const int64_t target = 148 * 4;
    int64_t chr = (total_rows + target - 1) / target;
    chr = std::min<int64_t>(16384, std::max<int64_t>(1024, (chr + 127) / 128 * 128));   // whole 128-row blocks
    // items <= rows / chr + anchor splits + one per tile; an item cut at the anchor limit spans
    // >= kSxAnc - 7 anchor slots (it is cut at a whole atom, and an atom spans <= 8 slots)
    static_assert(kSxAnc >= 8, "items must span whole atoms");
    const int64_t items_max = (total_rows + chr - 1) / chr + total_slots / (kSxAnc - 7) + ntiles + 1;
    const size_t ir0_bytes = ((size_t)items_max * 8 + 255) & ~size_t(255);
    rowbuf.ensure(rinfo_bytes + ktab_bytes + slot_bytes + ir0_bytes);
    uint4* ri = use_tc ? reinterpret_cast<uint4*>(rowbuf.as<char>()) : nullptr;
    float* ktab = reinterpret_cast<float*>(rowbuf.as<char>() + rinfo_bytes);
    uint32_t* slot_anchor = reinterpret_cast<uint32_t*>(rowbuf.as<char>() + rinfo_bytes + ktab_bytes);
    int64_t* item_r0 = reinterpret_cast<int64_t*>(rowbuf.as<char>() + rinfo_bytes + ktab_bytes + slot_bytes);
    if (use_f16 && ntiles > 0) {
        k_expand_atoms<<<(unsigned)ntiles, 256, 0, s>>>(segbuf.as<Seg>(), nseg, segcap, rows_off, aoff, a.rgrp, ri,
                                                        slot_anchor);
        BLSH_LAUNCH_CHECK();
        ++*launches;
    } else if (use_tc && ntiles > 0) {
        BLSH_CUDA(cudaMemsetAsync(aoff, 0, (size_t)(ntiles + 1) * 8, s));
        k_expand_rows<<<(unsigned)ntiles, 256, 0, s>>>(segbuf.as<Seg>(), nseg, segcap, rows_off, aoff, ri, nullptr,
                                                       nullptr);
        BLSH_LAUNCH_CHECK();
        ++*launches;
    }
    const unsigned gt = (unsigned)((ntiles + 255) / 256);
    const uint4* ri_split = use_f16 ? ri : nullptr;
    k_tile_items<<<gt, 256, 0, s>>>(wrows, rows_off, ri_split, ntiles, (int)chr, kSxAnc, items, nullptr, nullptr);
    BLSH_LAUNCH_CHECK();
    scan_exclusive_i64(items, item_off, ntiles, scan, s);
    k_tile_items<<<gt, 256, 0, s>>>(wrows, rows_off, ri_split, ntiles, (int)chr, kSxAnc, items, item_off, item_r0);
    BLSH_LAUNCH_CHECK();
    *launches += 5;
    int64_t n_items = 0;
    BLSH_CUDA(cudaMemcpyAsync(&n_items, item_off + ntiles, 8, cudaMemcpyDeviceToHost, s));
    BLSH_CUDA(cudaStreamSynchronize(s));
    const int nlist = use_f16 ? kSxEpiN : 4;   // buffered-pair lists per (item, query): the screen's epilogue warps
    const bool large_k = k > 64;               // fp16 screen + exact keys per query + launch_select
    // large k: each warp's list holds ~kk = ceil(k/8) survivors (+ the bound's slack)
    // fp16 screen: buffered pairs per (item, query, epilogue warp): 384.  A list that overflows
    // sends every row of its unit to exact rescoring, by one warp: with 96 (k <= 64) c3 at k = 50
    // (58k candidates per query) overflowed 87k lists (207M exact pairs, 40 ms; 384: none, 8M,
    // 1.8 ms), c5 with Morton-curve probing T = 64 spent 8.6 ms on a few overflowed units, and the
    // large-k lists (2 kk + 64) overflowed on c3 at k = 500 (428M exact pairs, 76 ms) (r02ak,
    // r02ao).  The buffers are plain HBM (n_items x 32 x 8 x 384 x 8 B: 3.1 GB at c4); the TF32
    // screen keeps its 96.  BLSH_SCAPW overrides (experiments).
    static const int scap_env = [] {
        const char* e = std::getenv("BLSH_SCAPW");
        return e ? std::max(32, std::atoi(e) / 16 * 16) : 0;
    }();
    const int scapw = use_f16 ? (scap_env ? scap_env : 384) : kTcScap;
    const int kScap = nlist * scapw;
    const size_t part_bytes = large_k ? 0 : ((size_t)std::max<int64_t>(n_items, 1) * QT * k * 8 + 255) & ~size_t(255);
    const size_t sbuf_bytes = ((size_t)std::max<int64_t>(n_items, 1) * QT * kScap * 8 + 255) & ~size_t(255);
    const size_t ufin_bytes = ((size_t)std::max<int64_t>(n_items, 1) * QT * 4 + 255) & ~size_t(255);
    const size_t scnt_bytes = ((size_t)std::max<int64_t>(n_items, 1) * QT * nlist * 4 + 255) & ~size_t(255);
    // large k: unit counts, unit offsets in their query's segment, query counts, segment offsets
    const size_t unit_bytes = large_k ? (((size_t)std::max<int64_t>(n_items, 1) * QT * 8 + 255) & ~size_t(255)) : 0;
    const size_t q_bytes = large_k ? (((size_t)(nq + 1) * 8 + 255) & ~size_t(255)) : 0;
    partials.ensure(part_bytes + sbuf_bytes + ufin_bytes + scnt_bytes + 2 * unit_bytes + 2 * q_bytes);
    TiledArgs ta{};
    ta.nq = nq; ta.ntiles = ntiles; ta.n_items = n_items; ta.d = a.d; ta.ds = a.ds; ta.k = k; ta.chr = (int)chr;
    ta.segcap = segcap; ta.Q = a.Q; ta.Xp = Xp; ta.perm = perm; ta.qorder = qorder; ta.segs = segbuf.as<Seg>();
    ta.nseg = nseg; ta.rows = wrows; ta.item_off = item_off; ta.partials = partials.as<unsigned long long>();
    ta.counters = counters;
    ta.tile_off = tile_off;
    ta.tile_of = tile_of;
    ta.sbuf = reinterpret_cast<unsigned long long*>(partials.as<char>() + part_bytes);
    ta.scap = kScap;
    ta.scapw = scapw;
    ta.nlist = nlist;
    ta.rows_off = rows_off;
    ta.ufin = reinterpret_cast<uint32_t*>(partials.as<char>() + part_bytes + sbuf_bytes);
    ta.scnt = reinterpret_cast<int32_t*>(partials.as<char>() + part_bytes + sbuf_bytes + ufin_bytes);
    ta.item_r0 = item_r0;
    ta.rowinfo = ri;
    ta.anc = a.anc;
    ta.dr = a.dr;
    ta.Rh = reinterpret_cast<const __half*>(a.Rh);
    ta.natom = a.natom;
    ta.rconst = a.rconst;
    ta.ktab = ktab;
    ta.slot_anchor = slot_anchor;
    if (const char* dm = std::getenv("BLSH_TC_MODE")) ta.dbgmode = std::atoi(dm);
    const size_t smem = tiled_smem_bytes(a.ds);
    const int nst = use_f16 ? screen_stages(a.dr) : 0;
    const size_t tc_smem = use_f16 ? screen_smem_bytes(a.dr, nst) : tc_smem_bytes(a.ds);
    const char* dbg_path = std::getenv("BLSH_TC_DEBUG");
    DevBuf dbgbuf;
    constexpr int kDbgN = 4096 + 2048;
    if (use_tc && dbg_path) {
        dbgbuf.alloc(kDbgN * sizeof(float));
        BLSH_CUDA(cudaMemsetAsync(dbgbuf.p, 0, kDbgN * sizeof(float), s));
        ta.dbg = dbgbuf.as<float>();
    }
    DevBuf tsbuf;
    if (use_tc && (ta.dbgmode & 32) && n_items > 0) {
        tsbuf.alloc((size_t)n_items * 16 * 8);
        BLSH_CUDA(cudaMemsetAsync(tsbuf.p, 0, (size_t)n_items * 16 * 8, s));
        ta.tstamp = tsbuf.as<unsigned long long>();
    }
    if (use_f16 && total_slots > 0) {
        const size_t ks = (size_t)QT * (a.ds / 4 + 1) * sizeof(float4);
        BLSH_CUDA(cudaFuncSetAttribute(k_anchor_k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)ks));
        k_anchor_k<<<(unsigned)ntiles, 256, ks, s>>>(a.Q, a.ds, qorder, tile_off, aoff, slot_anchor, a.anc, a.dr, ktab);
        BLSH_LAUNCH_CHECK();
        ++*launches;
    }
    if (ev_sl0) BLSH_CUDA(cudaEventRecord(ev_sl0, s));
    if (n_items > 0) {
        if (use_f16) {
            auto pick = [&](auto k8, auto k12, auto k16, auto k32, auto k64) {   // k > 64: KT = 64 (kk lists)
                return k <= 8 ? k8 : (k <= 12 ? k12 : (k <= 16 ? k16 : (k <= 32 ? k32 : k64)));
            };
            auto kern = nst == 8 ? pick(k_screen_f16<8, 8>, k_screen_f16<12, 8>, k_screen_f16<16, 8>, k_screen_f16<32, 8>,
                                        k_screen_f16<64, 8>)
                      : nst == 6 ? pick(k_screen_f16<8, 6>, k_screen_f16<12, 6>, k_screen_f16<16, 6>, k_screen_f16<32, 6>,
                                        k_screen_f16<64, 6>)
                                 : pick(k_screen_f16<8, 4>, k_screen_f16<12, 4>, k_screen_f16<16, 4>, k_screen_f16<32, 4>,
                                        k_screen_f16<64, 4>);
            BLSH_CUDA(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)tc_smem));
            kern<<<(unsigned)n_items, kSxThreads, tc_smem, s>>>(ta);
        } else if (use_tc) {
            auto kern = k <= 8 ? k_shortlist_tc<8>
                      : (k <= 12 ? k_shortlist_tc<12> : (k <= 16 ? k_shortlist_tc<16> : k_shortlist_tc<32>));
            BLSH_CUDA(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)tc_smem));
            kern<<<(unsigned)n_items, kTcThreads, tc_smem, s>>>(ta);
        }
        if (use_tc && large_k) {
            BLSH_LAUNCH_CHECK();
            ++*launches;
            if (ev_mid) BLSH_CUDA(cudaEventRecord(ev_mid, s));
            char* pb = partials.as<char>() + part_bytes + sbuf_bytes + ufin_bytes + scnt_bytes;
            int64_t* ucnt = reinterpret_cast<int64_t*>(pb);
            int64_t* uloc = reinterpret_cast<int64_t*>(pb + unit_bytes);
            int64_t* qcnt = reinterpret_cast<int64_t*>(pb + 2 * unit_bytes);
            int64_t* coff = reinterpret_cast<int64_t*>(pb + 2 * unit_bytes + q_bytes);
            const unsigned rg = (unsigned)((n_items * QT + 7) / 8);
            BLSH_CUDA(cudaMemsetAsync(qcnt, 0, (size_t)nq * 8, s));
            k_unit_counts<<<rg, 256, 0, s>>>(ta, ucnt);
            BLSH_LAUNCH_CHECK();
            k_query_counts<<<(unsigned)((nq + 255) / 256), 256, 0, s>>>(ta, ucnt, uloc, qcnt);
            BLSH_LAUNCH_CHECK();
            scan_exclusive_i64(qcnt, coff, nq, scan, s);
            *launches += 5;
            int64_t nkeys = 0;
            BLSH_CUDA(cudaMemcpyAsync(&nkeys, coff + nq, 8, cudaMemcpyDeviceToHost, s));
            BLSH_CUDA(cudaStreamSynchronize(s));
            keybuf.ensure((size_t)std::max<int64_t>(nkeys, 1) * 8);
            unsigned long long* keys = keybuf.as<unsigned long long>();
            const int nvq = (a.ds / 4 + 31) / 32;
            if (nvq <= 1) k_tc_emit<1><<<rg, 256, 0, s>>>(ta, uloc, coff, keys);
            else if (nvq == 2) k_tc_emit<2><<<rg, 256, 0, s>>>(ta, uloc, coff, keys);
            else if (nvq == 3) k_tc_emit<3><<<rg, 256, 0, s>>>(ta, uloc, coff, keys);
            else k_tc_emit<4><<<rg, 256, 0, s>>>(ta, uloc, coff, keys);
            BLSH_LAUNCH_CHECK();
            ++*launches;
            if (ev_sl1) BLSH_CUDA(cudaEventRecord(ev_sl1, s));
            launch_select(keys, coff, nq, k, a.qoor, a.cnt, out_ids, out_d2, out_packed, out_ncand, s);
            *launches += 2;
        } else if (use_tc) {
            BLSH_LAUNCH_CHECK();
            ++*launches;
            if (ev_mid) BLSH_CUDA(cudaEventRecord(ev_mid, s));
            const unsigned rg = (unsigned)((n_items * QT + 7) / 8);
            const int nvq = (a.ds / 4 + 31) / 32;
            // (cp.async staging of the rescored rows, as in k_shortlist's interval mode, measured
            // slower here: 0.92 -> 1.09 ms at c4, the rows of a tile's queries overlap in L1/L2, r02au)
            if (nvq <= 1) k_tc_rescore<1><<<rg, 256, 0, s>>>(ta);
            else if (nvq == 2) k_tc_rescore<2><<<rg, 256, 0, s>>>(ta);
            else if (nvq == 3) k_tc_rescore<3><<<rg, 256, 0, s>>>(ta);
            else k_tc_rescore<4><<<rg, 256, 0, s>>>(ta);
        } else {
            BLSH_CUDA(cudaFuncSetAttribute(k_shortlist_tiled, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
            k_shortlist_tiled<<<(unsigned)n_items, kTiledThreads, smem, s>>>(ta);
        }
        BLSH_LAUNCH_CHECK();
        ++*launches;
    }
    if (ev_mid && !use_tc) BLSH_CUDA(cudaEventRecord(ev_mid, s));
    if (!(large_k && n_items > 0)) {
        if (ev_sl1) BLSH_CUDA(cudaEventRecord(ev_sl1, s));
        if (large_k) {   // no work item: padding only
            char* pb = partials.as<char>() + part_bytes + sbuf_bytes + ufin_bytes + scnt_bytes;
            int64_t* coff = reinterpret_cast<int64_t*>(pb + 2 * unit_bytes + q_bytes);
            BLSH_CUDA(cudaMemsetAsync(coff, 0, (size_t)(nq + 1) * 8, s));
            launch_select(keybuf.as<unsigned long long>(), coff, nq, k, a.qoor, a.cnt, out_ids, out_d2, out_packed,
                          out_ncand, s);
            *launches += 2;
        } else {
            k_merge_tiled<<<(unsigned)((nq + 7) / 8), 256, 0, s>>>(ta, a.qoor, a.cnt, out_ids, out_d2, out_packed,
                                                                   out_ncand);
            BLSH_LAUNCH_CHECK();
            ++*launches;
        }
    }
    *n_items_out = n_items;
    *chr_out = (int)chr;
    *rows_out = total_rows;
    unsigned long long ev[5] = {0, 0, 0, 0, 0};
    BLSH_CUDA(cudaMemcpyAsync(ev, counters, 40, cudaMemcpyDeviceToHost, s));
    BLSH_CUDA(cudaStreamSynchronize(s));
    *pairs_out = (int64_t)(use_tc ? ev[1] : ev[0]);   // TC: exact rescorings after the screen
    *kept_out = use_tc ? (int64_t)ev[0] : 0;
    *kslots_out = use_f16 ? total_slots : 0;
    *screen_kind_out = use_f16 ? 1 : (use_tc ? 2 : 0);
    // every work item loads its tile's queries: sum over tiles of |tile| x items(tile) ~ n_items x nq / ntiles
    *qload_rows_out = ntiles > 0 ? (double)n_items * (double)nq / (double)ntiles : 0.0;
    if (use_tc && std::getenv("BLSH_TC_MODE"))
        std::fprintf(stderr, "[tc] items %lld kept %llu rescored %llu rows %lld insertions %llu compactions %llu "
                     "overflowed %llu\n", (long long)n_items, ev[0], ev[1], (long long)total_rows, ev[2], ev[3], ev[4]);
    if (ta.tstamp) {   // mean phase durations over items (us)
        std::vector<unsigned long long> h((size_t)n_items * 16);
        BLSH_CUDA(cudaMemcpy(h.data(), ta.tstamp, h.size() * 8, cudaMemcpyDeviceToHost));
        double acc[16] = {0};
        for (int64_t i = 0; i < n_items; ++i) {
            for (int p = 1; p < 6; ++p)
                if (h[i * 16 + p]) acc[p] += (double)(h[i * 16 + p] - h[i * 16]) * 1e-3;
            for (int p = 6; p < 14; ++p) acc[p] += (double)h[i * 16 + p] / 1965.0;   // cycles -> us at 1965 MHz
        }
        std::fprintf(stderr, "[tc] per item, us after start: setup %.1f producers %.1f mma %.1f epilogue %.1f end %.1f; "
                     "waits (us): producers on aempty %.1f, mfull %.1f, mempty %.1f; mma on afull %.1f, tempty %.1f; "
                     "epilogue on tfull %.1f, meta %.1f; mma issue+commit %.1f\n",
                     acc[1] / n_items, acc[2] / n_items, acc[3] / n_items, acc[4] / n_items, acc[5] / n_items,
                     acc[6] / n_items, acc[10] / n_items, acc[11] / n_items, acc[7] / n_items, acc[8] / n_items,
                     acc[9] / n_items, acc[12] / n_items, acc[13] / n_items);
    }
    if (ta.dbg) {
        std::vector<float> h(kDbgN);
        BLSH_CUDA(cudaMemcpy(h.data(), ta.dbg, h.size() * sizeof(float), cudaMemcpyDeviceToHost));
        std::vector<uint32_t> q0(QT);
        BLSH_CUDA(cudaMemcpy(q0.data(), qorder, QT * sizeof(uint32_t), cudaMemcpyDeviceToHost));
        if (FILE* f = std::fopen(dbg_path, "wb")) {
            std::fwrite(h.data(), sizeof(float), h.size(), f);
            std::fwrite(q0.data(), sizeof(uint32_t), q0.size(), f);
            std::fclose(f);
        }
    }
}

}  // namespace blsh
