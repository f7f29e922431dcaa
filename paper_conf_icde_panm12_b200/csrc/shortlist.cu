// shortlist.cu -- a5, the short-list search ("the main
// bottleneck ... more than 95% of the overall running time"), and the top-k
// merges (per-query chunk merge; a6 multi-GPU list merge).
//
// Layout: the table rows X_perm are stored in bucket
// order, so every candidate interval of a query is one contiguous slab.  A
// work item is (query, chunk of <= CH candidates); one warp owns an item,
// keeps the query slice in registers (lane l holds float4 columns l, l+32, ..),
// streams the slab with coalesced 128-bit loads four rows at a time, reduces
// the per-lane partial sums with a butterfly (fp32 direct form, R22), and keeps
// a warp-distributed sorted top-k of packed (d^2 bits << 32 | id) keys (lane l
// holds entries l and l+32).  Results per item go to a private slot, so the
// outcome never depends on scheduling.
#include <algorithm>

#include "internal.cuh"
#include "query_kernels.cuh"

namespace blsh {

namespace {

constexpr int kSLWarps = 8;

struct TopK {
    unsigned long long e0, e1;
};

__device__ __forceinline__ unsigned long long topk_thr(const TopK& t, int k) {
    return __shfl_sync(BLSH_FULL, k <= 32 ? t.e0 : t.e1, (k - 1) & 31);
}

// Insert a warp-uniform key v (caller guarantees v < threshold).
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

// EMIT = false: register top-k per item (k <= 64) into a.partials.
// EMIT = true (large k, k > 64): the packed key of every candidate goes to
// a.cand_keys[a.cand_off[q] + c] (c = rank of the candidate in the query's
// candidate order); k_select then takes the k smallest per query.
// LIST = false: the candidates are the query's T+1 position intervals (L = 1).
// LIST = true (L > 1 tables): the candidates are the deduplicated position list
// a.list[a.list_off[q] ..] that k_union_tables wrote (ascending positions).
// The distance arithmetic is the same in every mode (R22), so the modes agree
// bit for bit.
constexpr int kRG = 4;   // rows per distance group (loads in flight per lane: kRG x NV float4)

template <int NV, bool EMIT, bool LIST>
__global__ void __launch_bounds__(kSLWarps * 32) k_shortlist(ShortlistArgs a) {
    const int lane = threadIdx.x & 31;
    extern __shared__ float4 sl_stage[];   // interval mode: [kSLWarps][kRG][NV][32], row loads in flight
    float4* stg = sl_stage + (size_t)(threadIdx.x >> 5) * kRG * NV * 32;
    // grid-stride over the work items (a warp takes the next item as soon as it is done:
    // items differ in length, and a block would otherwise hold its slot until its slowest warp ends)
    // (list mode; the interval mode keeps one item per warp: neighbouring items, which share
    // rows in L2, then run together)
    // (with the item count on the device -- small batches -- the grid is bounded and strides too)
    const int64_t n_items = a.n_items_dev ? *a.n_items_dev : a.n_items;
    for (int64_t item = blockIdx.x * (int64_t)kSLWarps + (threadIdx.x >> 5); item < n_items;
         item += (LIST || a.n_items_dev) ? (int64_t)gridDim.x * kSLWarps : n_items) {
    // query of this item: last q with item_off[q] <= item
    int64_t lo = 0, hi = a.nq;
    while (hi - lo > 1) {
        const int64_t mid = (lo + hi) >> 1;
        if (a.item_off[mid] <= item) lo = mid;
        else hi = mid;
    }
    const int64_t q = lo;
    const int64_t c0 = (item - a.item_off[q]) * a.chunk;
    const int64_t c1 = min(c0 + a.chunk, a.cnt[q]);
    const int nv = a.ds >> 2;
    float4 qv[NV];
    const float4* qrow = reinterpret_cast<const float4*>(a.Q + (size_t)q * a.ds);
#pragma unroll
    for (int u = 0; u < NV; ++u) {
        const int v = lane + 32 * u;
        qv[u] = v < nv ? qrow[v] : make_float4(0.f, 0.f, 0.f, 0.f);
    }
    TopK tk{kEmpty, kEmpty};
    const int k = a.k;
    unsigned long long thr = kEmpty;
    // Rows r[0..nr) (table positions) that are candidates c, c+1, .. of q.
    auto group = [&](const int64_t (&r)[kRG], int nr, int64_t c) {
        float part[kRG];
        if constexpr (!LIST) {
            // interval mode (rows streamed once, the no-reuse regime): the group's kRG x NV 16-byte
            // loads in flight together, by cp.async into this warp's staging slots [j][u][lane],
            // one wait, then the chains read the lane's own slots (register loads: the compiler
            // consumed each row before issuing the next, 3 LDG.128 in flight per lane; c5 with
            // tiles off 0.79 -> 0.98 of measured HBM, r02au)
#pragma unroll
            for (int j = 0; j < kRG; ++j) {
                if (j < nr) {
                    const float4* xr = reinterpret_cast<const float4*>(a.Xp + (size_t)r[j] * a.ds);
#pragma unroll
                    for (int u = 0; u < NV; ++u) {
                        const int v = lane + 32 * u;
                        if (v < nv) {
                            const uint32_t dst = (uint32_t)__cvta_generic_to_shared(stg + (j * NV + u) * 32 + lane);
                            asm volatile("cp.async.ca.shared.global [%0], [%1], 16;" ::"r"(dst), "l"(xr + v) : "memory");
                        }
                    }
                }
            }
            asm volatile("cp.async.commit_group;\n\tcp.async.wait_group 0;" ::: "memory");
#pragma unroll
            for (int j = 0; j < kRG; ++j) {
                part[j] = 0.0f;
#pragma unroll
                for (int u = 0; u < NV; ++u) {
                    const int v = lane + 32 * u;
                    if (v < nv) {
                        const float4 x = stg[(j * NV + u) * 32 + lane];
                        float dx = qv[u].x - x.x, dy = qv[u].y - x.y, dz = qv[u].z - x.z, dw = qv[u].w - x.w;
                        part[j] = fmaf(dx, dx, part[j]);
                        part[j] = fmaf(dy, dy, part[j]);
                        part[j] = fmaf(dz, dz, part[j]);
                        part[j] = fmaf(dw, dw, part[j]);
                    }
                }
            }
        } else {
            // list mode (L > 1 tables, the E8 node: rows gathered, many served from L2): register
            // loads, which the compiler overlaps with the previous row's chain (the staging's
            // issue-then-wait measured slower here: p217 13.0 -> 17.3 ms, r02au)
#pragma unroll
            for (int j = 0; j < kRG; ++j) {
                part[j] = 0.0f;
                if (j < nr) {
                    const float4* xr = reinterpret_cast<const float4*>(a.Xp + (size_t)r[j] * a.ds);
#pragma unroll
                    for (int u = 0; u < NV; ++u) {
                        const int v = lane + 32 * u;
                        if (v < nv) {
                            const float4 x = __ldg(xr + v);
                            float dx = qv[u].x - x.x, dy = qv[u].y - x.y, dz = qv[u].z - x.z, dw = qv[u].w - x.w;
                            part[j] = fmaf(dx, dx, part[j]);
                            part[j] = fmaf(dy, dy, part[j]);
                            part[j] = fmaf(dz, dz, part[j]);
                            part[j] = fmaf(dw, dw, part[j]);
                        }
                    }
                }
            }
        }
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) {
#pragma unroll
            for (int j = 0; j < kRG; ++j) part[j] += __shfl_xor_sync(BLSH_FULL, part[j], o);
        }
        int64_t rl = r[0];
#pragma unroll
        for (int j = 1; j < kRG; ++j) rl = lane == j ? r[j] : rl;
        const uint32_t idl = (lane < nr) ? __ldg(a.perm + rl) : 0u;
        if (EMIT) {
            if (lane < nr) {
                float pj = part[0];
#pragma unroll
                for (int j = 1; j < kRG; ++j) pj = lane == j ? part[j] : pj;
                a.cand_keys[a.cand_off[q] + c + lane] = pack_entry(pj, idl);
            }
            return;
        }
#pragma unroll
        for (int j = 0; j < kRG; ++j) {
            const uint32_t id = __shfl_sync(BLSH_FULL, idl, j);
            if (j < nr) {
                const unsigned long long key = pack_entry(part[j], id);
                if (key < thr) {
                    topk_insert(tk, key, lane);
                    thr = topk_thr(tk, k);
                }
            }
        }
    };
    if (LIST) {
        const uint32_t* L = a.list + a.list_off[q];
        for (int64_t c = c0; c < c1; c += kRG) {
            const int nr = (int)min((int64_t)kRG, c1 - c);
            int64_t r[kRG];
#pragma unroll
            for (int j = 0; j < kRG; ++j) r[j] = j < nr ? (int64_t)__ldg(L + c + j) : 0;
            group(r, nr, c);
        }
    } else {
        const uint2* ivl = a.ivl + (size_t)q * (a.T + 1);
        int64_t acc = 0;   // candidates before the current interval
        for (int p = 0; p <= a.T && acc < c1; ++p) {
            const uint2 iv = ivl[p];
            const int64_t len = (int64_t)iv.y - (int64_t)iv.x;
            if (len <= 0) continue;
            const int64_t s = max(c0, acc), e = min(c1, acc + len);
            if (s < e) {
                const int64_t pa = (int64_t)iv.x + (s - acc), pb = (int64_t)iv.x + (e - acc);
                for (int64_t r0 = pa; r0 < pb; r0 += kRG) {
                    const int nr = (int)min((int64_t)kRG, pb - r0);
                    int64_t r[kRG];
#pragma unroll
                    for (int j = 0; j < kRG; ++j) r[j] = r0 + j;
                    group(r, nr, acc + (r0 - (int64_t)iv.x));
                }
            }
            acc += len;
        }
    }
    if (!EMIT) {
        unsigned long long* out = a.partials + (size_t)item * k;
        if (lane < k) out[lane] = tk.e0;
        if (lane + 32 < k) out[lane + 32] = tk.e1;
    }
    }   // item loop
}

__global__ void k_items(const int64_t* __restrict__ cnt, int64_t nq, int chunk, int64_t* __restrict__ items) {
    const int64_t q = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (q < nq) items[q] = (cnt[q] + chunk - 1) / chunk;
}

__device__ __forceinline__ void write_out(const TopK& tk, int64_t q, int k, int lane, int64_t* out_ids,
                                          float* out_d2, unsigned long long* out_packed) {
#pragma unroll
    for (int h = 0; h < 2; ++h) {
        const int i = lane + 32 * h;
        if (i >= k) continue;
        const unsigned long long e = h ? tk.e1 : tk.e0;
        if (out_packed) out_packed[(size_t)q * k + i] = e == kEmpty ? kPadPacked : e;
        if (out_ids) out_ids[(size_t)q * k + i] = e == kEmpty ? -1 : (int64_t)(uint32_t)(e & 0xFFFFFFFFull);
        if (out_d2) out_d2[(size_t)q * k + i] = e == kEmpty ? __int_as_float(0x7F800000) : __uint_as_float((uint32_t)(e >> 32));
    }
}

// Per query: merge the sorted partial lists of its items.
__global__ void __launch_bounds__(256) k_merge(ShortlistArgs a, const int32_t* __restrict__ qoor, int64_t* out_ids,
                                               float* out_d2, unsigned long long* out_packed, int64_t* out_ncand) {
    const int lane = threadIdx.x & 31;
    const int64_t q = blockIdx.x * (int64_t)(blockDim.x >> 5) + (threadIdx.x >> 5);
    if (q >= a.nq) return;
    const int k = a.k;
    TopK tk{kEmpty, kEmpty};
    unsigned long long thr = kEmpty;
    const int64_t it0 = a.item_off[q], it1 = a.item_off[q + 1];
    auto load = [&](int64_t it, unsigned long long& l0, unsigned long long& l1) {
        const unsigned long long* L = a.partials + (size_t)it * k;
        l0 = lane < k ? L[lane] : kEmpty;
        l1 = lane + 32 < k ? L[lane + 32] : kEmpty;
    };
    unsigned long long c0 = kEmpty, c1 = kEmpty;
    if (it0 < it1) load(it0, c0, c1);
    for (int64_t it = it0; it < it1; ++it) {
        unsigned long long n0 = kEmpty, n1 = kEmpty;
        if (it + 1 < it1) load(it + 1, n0, n1);   // the next list is in flight during this one's inserts
        for (int j = 0; j < k; ++j) {
            const unsigned long long v = __shfl_sync(BLSH_FULL, j < 32 ? c0 : c1, j & 31);
            if (v >= thr) break;
            topk_insert(tk, v, lane);
            thr = topk_thr(tk, k);
        }
        c0 = n0;
        c1 = n1;
    }
    write_out(tk, q, k, lane, out_ids, out_d2, out_packed);
    if (lane == 0 && out_ncand) out_ncand[q] = (qoor[q] & 2) ? 0 : a.cnt[q];
}

// a6: per query, k smallest over n_lists packed lists [n_lists][nq][k].
__global__ void __launch_bounds__(256) k_merge_lists(const unsigned long long* __restrict__ packed, int n_lists,
                                                     int64_t nq, int k, int64_t* out_ids, float* out_d2) {
    const int lane = threadIdx.x & 31;
    const int64_t q = blockIdx.x * (int64_t)(blockDim.x >> 5) + (threadIdx.x >> 5);
    if (q >= nq) return;
    TopK tk{kEmpty, kEmpty};
    unsigned long long thr = kEmpty;
    for (int l = 0; l < n_lists; ++l) {
        const unsigned long long* L = packed + ((size_t)l * nq + q) * k;
        const unsigned long long l0 = lane < k ? L[lane] : kEmpty;
        const unsigned long long l1 = lane + 32 < k ? L[lane + 32] : kEmpty;
        for (int j = 0; j < k; ++j) {
            unsigned long long v = __shfl_sync(BLSH_FULL, j < 32 ? l0 : l1, j & 31);
            if (v == kPadPacked) v = kEmpty;
            if (v >= thr) break;
            topk_insert(tk, v, lane);
            thr = topk_thr(tk, k);
        }
    }
    write_out(tk, q, k, lane, out_ids, out_d2, nullptr);
}

// ---- large k (64 < k <= 1024): block radix select -------------------------------
// One CTA per query selects the k smallest packed keys of the query's segment
// (the candidate keys k_shortlist<.., true> emitted, or for the a6 merge the
// n_lists sorted lists of k entries) and writes them in ascending order.  Keys
// of distinct candidates are distinct (ids are); only padding repeats, and
// padding is larger than every real key.
//   MSB-first radix select, 8 bits per pass: histogram of the current byte over
//   the keys that match the prefix so far, pick the bin holding the need-th
//   key; stop early when that bin is taken whole.  Then the selected keys
//   (<= k) are collected into shared memory and bitonic-sorted.
constexpr int kSelThreads = 512;
constexpr int kSmallSel = 512;  // queries with at most this many candidates: warp-register sort
constexpr int kSelCap = 1024;   // max k

struct SelSrc {
    const unsigned long long* base;
    int64_t off, len;      // segment mode: keys base[off .. off+len)
    int n_lists;           // list mode (n_lists > 0): list l entries at base[(l*nq + q)*k + j]
    int64_t nq, q;
    int k;
    __device__ __forceinline__ unsigned long long get(int64_t i) const {
        if (n_lists == 0) return base[off + i];
        const int64_t l = i / k, j = i - l * k;
        const unsigned long long v = base[((size_t)l * nq + q) * k + j];
        return v == kPadPacked ? kEmpty : v;
    }
};

__device__ void block_select_write(const SelSrc& src, int k, int64_t q, int64_t* out_ids, float* out_d2,
                                   unsigned long long* out_packed) {
    __shared__ unsigned int hist[256];
    __shared__ unsigned long long buf[kSelCap];
    __shared__ unsigned long long s_prefix, s_mask;
    __shared__ int s_need, s_whole, s_cnt;
    const int tid = threadIdx.x;
    const int64_t len = src.len;
    unsigned long long thr_le;   // keys <= thr_le are all taken
    int fill_eq = 0;             // ... plus fill_eq copies of thr_eq
    unsigned long long thr_eq = kEmpty;
    if (len <= k) {
        thr_le = kEmpty;
    } else {
        if (tid == 0) { s_prefix = 0; s_mask = 0; s_need = k; s_whole = 0; }
        __syncthreads();
        for (int byte = 7; byte >= 0; --byte) {
            for (int i = tid; i < 256; i += kSelThreads) hist[i] = 0;
            __syncthreads();
            const unsigned long long pre = s_prefix, msk = s_mask;
            const int sh = byte * 8;
            for (int64_t i = tid; i < len; i += kSelThreads) {
                const unsigned long long v = src.get(i);
                if ((v & msk) == pre) atomicAdd(&hist[(v >> sh) & 255], 1u);
            }
            __syncthreads();
            if (tid < 32) {   // warp 0: find the bin of the need-th key
                const int need = s_need;
                unsigned int c[8], tot = 0;
#pragma unroll
                for (int j = 0; j < 8; ++j) { c[j] = hist[tid * 8 + j]; tot += c[j]; }
                unsigned int incl = tot;
#pragma unroll
                for (int o = 1; o < 32; o <<= 1) {
                    const unsigned int t = __shfl_up_sync(BLSH_FULL, incl, o);
                    if (tid >= o) incl += t;
                }
                const unsigned int excl = incl - tot;
                const bool mine = excl < (unsigned)need && (unsigned)need <= incl;
                if (mine) {
                    unsigned int run = excl;
                    int bin = tid * 8;
#pragma unroll
                    for (int j = 0; j < 8; ++j) {
                        if (run + c[j] >= (unsigned)need) { bin = tid * 8 + j; break; }
                        run += c[j];
                    }
                    const unsigned int inbin = hist[bin];
                    s_need = need - (int)run;
                    s_prefix = pre | ((unsigned long long)bin << sh);
                    s_mask = msk | (255ull << sh);
                    s_whole = (run + inbin == (unsigned)need) ? 1 : 0;
                }
            }
            __syncthreads();
            if (s_whole) break;
        }
        if (s_whole) {
            thr_le = s_prefix | ~s_mask;          // exactly k keys are <= this
        } else {
            thr_eq = s_prefix;                    // the k-th key, repeated s_need times at the cut
            fill_eq = s_need;
            thr_le = thr_eq - 1;                  // keys strictly below it
            if (thr_eq == 0) { thr_le = 0; fill_eq = 0; }
        }
    }
    __syncthreads();
    if (tid == 0) s_cnt = 0;
    for (int i = tid; i < kSelCap; i += kSelThreads) buf[i] = kEmpty;   // (only the sorted prefix is read)
    __syncthreads();
    const bool take_all = len <= k;
    if (take_all) {   // every key is selected: position = index, no counter
        for (int64_t i = tid; i < len; i += kSelThreads) buf[i] = src.get(i);
        if (tid == 0) s_cnt = (int)len;
    } else {          // warp-aggregated slots: one shared atomic per warp and pass
        const int lane = tid & 31;
        for (int64_t b0 = 0; b0 < len; b0 += kSelThreads) {
            const int64_t i = b0 + tid;
            const unsigned long long v = i < len ? src.get(i) : kEmpty;
            const bool take = i < len && v <= thr_le;
            const unsigned m = __ballot_sync(BLSH_FULL, take);
            int base = 0;
            if (lane == 0 && m) base = atomicAdd(&s_cnt, __popc(m));
            base = __shfl_sync(BLSH_FULL, base, 0);
            if (take) {
                const int slot = base + __popc(m & lanemask_lt());
                if (slot < kSelCap) buf[slot] = v;
            }
        }
    }
    __syncthreads();
    if (fill_eq > 0) {
        const int base = s_cnt;
        for (int i = tid; i < fill_eq; i += kSelThreads)
            if (base + i < kSelCap) buf[base + i] = thr_eq;
        __syncthreads();
    }
    // bitonic sort of the first npow keys (npow = the power of two >= the selected
    // count, >= 64; padding kEmpty sorts last)
    const int nsel = (int)min((int64_t)k, len);
    int npow = 64;
    while (npow < nsel) npow <<= 1;
    for (int size = 2; size <= npow; size <<= 1) {
        for (int stride = size >> 1; stride > 0; stride >>= 1) {
            for (int i = tid; i < npow / 2; i += kSelThreads) {
                const int lo = 2 * i - (i & (stride - 1));
                const int hi = lo + stride;
                const bool up = (lo & size) == 0;
                const unsigned long long x = buf[lo], y = buf[hi];
                if ((x > y) == up) { buf[lo] = y; buf[hi] = x; }
            }
            __syncthreads();
        }
    }
    for (int i = tid; i < k; i += kSelThreads) {
        const unsigned long long e = buf[i];
        if (out_packed) out_packed[(size_t)q * k + i] = e == kEmpty ? kPadPacked : e;
        if (out_ids) out_ids[(size_t)q * k + i] = e == kEmpty ? -1 : (int64_t)(uint32_t)(e & 0xFFFFFFFFull);
        if (out_d2) out_d2[(size_t)q * k + i] = e == kEmpty ? __int_as_float(0x7F800000) : __uint_as_float((uint32_t)(e >> 32));
    }
}

// a5, large k: per query, the k smallest of its emitted candidate keys.
__global__ void __launch_bounds__(kSelThreads) k_select(const unsigned long long* __restrict__ cand_keys,
                                                        const int64_t* __restrict__ cand_off, int64_t nq, int k,
                                                        const int32_t* __restrict__ qoor, const int64_t* __restrict__ cnt,
                                                        int64_t* out_ids, float* out_d2, unsigned long long* out_packed,
                                                        int64_t* out_ncand) {
    const int64_t q = blockIdx.x;
    if (cand_off[q + 1] - cand_off[q] <= kSmallSel) return;   // k_select_small's query
    SelSrc src{cand_keys, cand_off[q], cand_off[q + 1] - cand_off[q], 0, nq, q, k};
    block_select_write(src, k, q, out_ids, out_d2, out_packed);
    if (threadIdx.x == 0 && out_ncand) out_ncand[q] = (qoor[q] & 2) ? 0 : cnt[q];
}

// a5, large k, queries with <= 512 candidates (all of them are in the answer or the
// answer is their sorted prefix): one warp per query sorts its keys in registers -- key
// i = 32 r + lane in v[r]; bitonic strides < 32 by shuffles, >= 32 between a lane's own
// registers -- no shared memory, no barriers.
__global__ void __launch_bounds__(256) k_select_small(const unsigned long long* __restrict__ cand_keys,
                                                      const int64_t* __restrict__ cand_off, int64_t nq, int k,
                                                      const int32_t* __restrict__ qoor, const int64_t* __restrict__ cnt,
                                                      int64_t* out_ids, float* out_d2, unsigned long long* out_packed,
                                                      int64_t* out_ncand) {
    constexpr int R = kSmallSel / 32;   // keys per lane
    const int lane = threadIdx.x & 31;
    const int64_t q = blockIdx.x * (int64_t)(blockDim.x >> 5) + (threadIdx.x >> 5);
    if (q >= nq) return;
    const int64_t off = cand_off[q], len = cand_off[q + 1] - off;
    if (len > kSmallSel) return;        // k_select's query
    unsigned long long v[R];
#pragma unroll
    for (int r = 0; r < R; ++r) {
        const int i = 32 * r + lane;
        v[r] = i < len ? cand_keys[off + i] : kEmpty;
    }
#pragma unroll
    for (int size = 2; size <= kSmallSel; size <<= 1) {
#pragma unroll
        for (int stride = size >> 1; stride > 0; stride >>= 1) {
            if (stride >= 32) {
                const int rs = stride >> 5;
#pragma unroll
                for (int r = 0; r < R; ++r) {
                    if (r & rs) continue;   // (r, r | rs): the lower index keeps the min when ascending
                    const int i = 32 * r + lane;
                    const bool up = (i & size) == 0;
                    const unsigned long long x = v[r], y = v[r | rs];
                    const bool sw = (x > y) == up;
                    v[r] = sw ? y : x;
                    v[r | rs] = sw ? x : y;
                }
            } else {
#pragma unroll
                for (int r = 0; r < R; ++r) {
                    const unsigned long long o = __shfl_xor_sync(BLSH_FULL, v[r], stride);
                    const int i = 32 * r + lane;
                    const bool take_min = ((lane & stride) == 0) == ((i & size) == 0);
                    v[r] = take_min ? (v[r] < o ? v[r] : o) : (v[r] < o ? o : v[r]);
                }
            }
        }
    }
#pragma unroll
    for (int r = 0; r < R; ++r) {
        const int i = 32 * r + lane;
        if (i < k) {
            const unsigned long long e = v[r];
            if (out_packed) out_packed[(size_t)q * k + i] = e == kEmpty ? kPadPacked : e;
            if (out_ids) out_ids[(size_t)q * k + i] = e == kEmpty ? -1 : (int64_t)(uint32_t)(e & 0xFFFFFFFFull);
            if (out_d2) out_d2[(size_t)q * k + i] = e == kEmpty ? __int_as_float(0x7F800000) : __uint_as_float((uint32_t)(e >> 32));
        }
    }
    for (int i = kSmallSel + lane; i < k; i += 32) {   // k > 512: padding beyond the sorted keys
        if (out_packed) out_packed[(size_t)q * k + i] = kPadPacked;
        if (out_ids) out_ids[(size_t)q * k + i] = -1;
        if (out_d2) out_d2[(size_t)q * k + i] = __int_as_float(0x7F800000);
    }
    if (lane == 0 && out_ncand) out_ncand[q] = (qoor[q] & 2) ? 0 : cnt[q];
}

// a6, large k: per query, the k smallest over n_lists packed lists.
__global__ void __launch_bounds__(kSelThreads) k_select_lists(const unsigned long long* __restrict__ packed,
                                                              int n_lists, int64_t nq, int k, int64_t* out_ids,
                                                              float* out_d2) {
    const int64_t q = blockIdx.x;
    SelSrc src{packed, 0, (int64_t)n_lists * k, n_lists, nq, q, k};
    block_select_write(src, k, q, out_ids, out_d2, nullptr);
}

}  // namespace

void launch_items(const int64_t* cnt, int64_t nq, int chunk, int64_t* items, cudaStream_t s) {
    if (nq == 0) return;
    k_items<<<(unsigned)((nq + 255) / 256), 256, 0, s>>>(cnt, nq, chunk, items);
    BLSH_LAUNCH_CHECK();
}

void launch_shortlist(const ShortlistArgs& a, cudaStream_t s) {
    if (a.n_items == 0) return;
    const int64_t blocks = (a.n_items + kSLWarps - 1) / kSLWarps;
    const unsigned grid = (unsigned)((a.list || a.n_items_dev) ? std::min<int64_t>(blocks, 148 * 8) : blocks);
    const int nvl = ((a.ds >> 2) + 31) / 32;

    const int smem = a.list ? 0 : kSLWarps * kRG * nvl * 32 * 16;   // interval mode stages its row loads
    auto go = [&](auto kern) {
        if (smem > 48 * 1024) BLSH_CUDA(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
        kern<<<grid, kSLWarps * 32, smem, s>>>(a);
    };
#define BLSH_SL_CASE(V)                                                                             \
    case V:                                                                                         \
        if (a.list) {                                                                               \
            if (a.cand_keys) go(k_shortlist<V, true, true>);                                        \
            else go(k_shortlist<V, false, true>);                                                   \
        } else {                                                                                    \
            if (a.cand_keys) go(k_shortlist<V, true, false>);                                       \
            else go(k_shortlist<V, false, false>);                                                  \
        }                                                                                           \
        break;
    switch (nvl) {
        BLSH_SL_CASE(1) BLSH_SL_CASE(2) BLSH_SL_CASE(3) BLSH_SL_CASE(4)
        BLSH_SL_CASE(5) BLSH_SL_CASE(6) BLSH_SL_CASE(7) BLSH_SL_CASE(8)
        default: throw Error(BLSH_ERR_UNSUPPORTED, "d > 1024");
    }
#undef BLSH_SL_CASE
    BLSH_LAUNCH_CHECK();
}

void launch_merge(const ShortlistArgs& a, const int32_t* qoor, int64_t* out_ids, float* out_d2,
                  unsigned long long* out_packed, int64_t* out_ncand, cudaStream_t s) {
    if (a.nq == 0) return;
    k_merge<<<(unsigned)((a.nq + 7) / 8), 256, 0, s>>>(a, qoor, out_ids, out_d2, out_packed, out_ncand);
    BLSH_LAUNCH_CHECK();
}

void merge_lists(const unsigned long long* packed, int n_lists, int64_t nq, int k, int64_t* out_ids,
                 float* out_d2, cudaStream_t s) {
    if (nq == 0) return;
    if (k > 64) {
        k_select_lists<<<(unsigned)nq, kSelThreads, 0, s>>>(packed, n_lists, nq, k, out_ids, out_d2);
        BLSH_LAUNCH_CHECK();
        return;
    }
    k_merge_lists<<<(unsigned)((nq + 7) / 8), 256, 0, s>>>(packed, n_lists, nq, k, out_ids, out_d2);
    BLSH_LAUNCH_CHECK();
}

void launch_select(const unsigned long long* cand_keys, const int64_t* cand_off, int64_t nq, int k,
                   const int32_t* qoor, const int64_t* cnt, int64_t* out_ids, float* out_d2,
                   unsigned long long* out_packed, int64_t* out_ncand, cudaStream_t s) {
    if (nq == 0) return;
    if (k > kSelCap) throw Error(BLSH_ERR_UNSUPPORTED, "k > 1024");
    k_select_small<<<(unsigned)((nq + 7) / 8), 256, 0, s>>>(cand_keys, cand_off, nq, k, qoor, cnt, out_ids, out_d2,
                                                             out_packed, out_ncand);
    BLSH_LAUNCH_CHECK();
    k_select<<<(unsigned)nq, kSelThreads, 0, s>>>(cand_keys, cand_off, nq, k, qoor, cnt, out_ids, out_d2, out_packed,
                                                  out_ncand);
    BLSH_LAUNCH_CHECK();
}

}  // namespace blsh
