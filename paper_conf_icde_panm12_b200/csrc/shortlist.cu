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

template <int NV>
__global__ void __launch_bounds__(kSLWarps * 32) k_shortlist(ShortlistArgs a) {
    const int lane = threadIdx.x & 31;
    const int64_t item = blockIdx.x * (int64_t)kSLWarps + (threadIdx.x >> 5);
    if (item >= a.n_items) return;
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
    const uint2* ivl = a.ivl + (size_t)q * (a.T + 1);
    int64_t acc = 0;   // candidates before the current interval
    for (int p = 0; p <= a.T && acc < c1; ++p) {
        const uint2 iv = ivl[p];
        const int64_t len = (int64_t)iv.y - (int64_t)iv.x;
        if (len <= 0) continue;
        const int64_t s = max(c0, acc), e = min(c1, acc + len);
        if (s < e) {
            const int64_t pa = (int64_t)iv.x + (s - acc), pb = (int64_t)iv.x + (e - acc);
            for (int64_t r0 = pa; r0 < pb; r0 += 4) {
                float part[4];
#pragma unroll
                for (int j = 0; j < 4; ++j) {
                    part[j] = 0.0f;
                    if (r0 + j < pb) {
                        const float4* xr = reinterpret_cast<const float4*>(a.Xp + (size_t)(r0 + j) * a.ds);
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
#pragma unroll
                for (int o = 16; o > 0; o >>= 1) {
#pragma unroll
                    for (int j = 0; j < 4; ++j) part[j] += __shfl_xor_sync(BLSH_FULL, part[j], o);
                }
                const uint32_t idl = (lane < 4 && r0 + lane < pb) ? __ldg(a.perm + r0 + lane) : 0u;
#pragma unroll
                for (int j = 0; j < 4; ++j) {
                    const uint32_t id = __shfl_sync(BLSH_FULL, idl, j);
                    if (r0 + j < pb) {
                        const unsigned long long key = pack_entry(part[j], id);
                        if (key < thr) {
                            topk_insert(tk, key, lane);
                            thr = topk_thr(tk, k);
                        }
                    }
                }
            }
        }
        acc += len;
    }
    unsigned long long* out = a.partials + (size_t)item * k;
    if (lane < k) out[lane] = tk.e0;
    if (lane + 32 < k) out[lane + 32] = tk.e1;
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
    for (int64_t it = a.item_off[q]; it < a.item_off[q + 1]; ++it) {
        const unsigned long long* L = a.partials + (size_t)it * k;
        const unsigned long long l0 = lane < k ? L[lane] : kEmpty;
        const unsigned long long l1 = lane + 32 < k ? L[lane + 32] : kEmpty;
        for (int j = 0; j < k; ++j) {
            const unsigned long long v = __shfl_sync(BLSH_FULL, j < 32 ? l0 : l1, j & 31);
            if (v >= thr) break;
            topk_insert(tk, v, lane);
            thr = topk_thr(tk, k);
        }
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

}  // namespace

void launch_items(const int64_t* cnt, int64_t nq, int chunk, int64_t* items, cudaStream_t s) {
    if (nq == 0) return;
    k_items<<<(unsigned)((nq + 255) / 256), 256, 0, s>>>(cnt, nq, chunk, items);
    BLSH_LAUNCH_CHECK();
}

void launch_shortlist(const ShortlistArgs& a, cudaStream_t s) {
    if (a.n_items == 0) return;
    const unsigned grid = (unsigned)((a.n_items + kSLWarps - 1) / kSLWarps);
    const int nvl = ((a.ds >> 2) + 31) / 32;
    switch (nvl) {
        case 1: k_shortlist<1><<<grid, kSLWarps * 32, 0, s>>>(a); break;
        case 2: k_shortlist<2><<<grid, kSLWarps * 32, 0, s>>>(a); break;
        case 3: k_shortlist<3><<<grid, kSLWarps * 32, 0, s>>>(a); break;
        case 4: k_shortlist<4><<<grid, kSLWarps * 32, 0, s>>>(a); break;
        case 5: k_shortlist<5><<<grid, kSLWarps * 32, 0, s>>>(a); break;
        case 6: k_shortlist<6><<<grid, kSLWarps * 32, 0, s>>>(a); break;
        case 7: k_shortlist<7><<<grid, kSLWarps * 32, 0, s>>>(a); break;
        case 8: k_shortlist<8><<<grid, kSLWarps * 32, 0, s>>>(a); break;
        default: throw Error(BLSH_ERR_UNSUPPORTED, "d > 1024");
    }
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
    k_merge_lists<<<(unsigned)((nq + 7) / 8), 256, 0, s>>>(packed, n_lists, nq, k, out_ids, out_d2);
    BLSH_LAUNCH_CHECK();
}

}  // namespace blsh
