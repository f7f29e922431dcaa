// query.cu -- a1-a4 of the query hot path.
//   k_route_hash   a1+a2: RP-tree routing + E2LSH projection (Eq. 2) /
//                  E8 decode (Eq. 6) + Morton key; canonical fp32 (R1).
//   k_probe_lookup a3+a4: probe sequence (standard, multiprobe P:247 / R11,
//                  E8 lattice P:147 / R15) and binary search of every probe key
//                  among the leaf's sorted bucket keys (R10); candidate
//                  intervals of the position-sorted table + |A0|.
//   k_median       tau = lower median of |A0| over the batch (R18).
//   k_widen        Morton-prefix widening until |R| >= tau (Eq. 7-8, R17).
#include <algorithm>
#include <array>
#include <mutex>
#include <vector>

#include "hashcore.cuh"
#include "internal.cuh"
#include "query_kernels.cuh"

namespace blsh {

__constant__ int8_t c_e8_roots[240][8];   // doubled coordinates, canonical order (R15)
__device__ int8_t g_e8_ring2[9120][8];     // recursive probing: the second ring, canonical order (R26)

namespace {

// ---------------------------------------------------------------------------
// a1 + a2
// ---------------------------------------------------------------------------
// Both passes read the query rows as 32-column chunks of 32 rows per warp, staged in
// shared memory with coalesced 16-byte loads (each row's 128-byte chunk is one line) and
// read back by lane = query (row pitch 36 floats: the 16-byte reads of 8 lanes fall in
// distinct bank groups).  A lane's chains stay canonical (R1: one fmaf per column, j
// strictly ascending from 0.0f); the chunking only changes where x_j comes from.
//   k_route_pass  ceil(depth / 3) passes; a pass evaluates the <= 7 nodes of the
//                 3-level subtree below the query's current node (independent chains:
//                 the FMA latency is hidden, the rows are read ceil(depth / 3) times
//                 instead of depth times), then descends 3 levels; between passes the
//                 queries are regrouped by the node reached, so a block's queries share
//                 their subtree and read its node vectors from shared memory.
//   k_leaf_scan / k_leaf_scatter   group the queries by leaf (lperm).
//   k_hash        128 leaf-grouped queries per block; the leaf matrix A_g of the
//                 block's first query is staged in shared memory (pitch ds, broadcast
//                 reads); each lane runs its M projection chains, Eq. 2 / E8, Morton key.
constexpr int kRHW = 4;              // warps per block (32 queries each)
constexpr int kRHQ = 32 * kRHW;      // queries per block
constexpr int kRHP = kRowPitch;      // staged chunk row pitch (floats, hashcore.cuh)

// One pass of a1 over levels [l0, l0 + 3): queries in `order` (NULL: batch order), grouped by
// the node they reached (qleaf holds its index within level l0; 0 at l0 = 0).  The block stages
// the 3-level subtree (<= 7 node vectors, dir or mu by the node's rule) below its first query's
// node in shared memory; a warp whose 32 queries all sit at that node reads it as broadcast
// 16-byte loads, other warps read their lanes' nodes through L1.  Every lane runs <= 7
// independent canonical chains (R1) over the row chunks, descends, and writes its node's index
// within level l0 + nl into qleaf, counted in cnt (the next grouping / the leaf histogram).
// PREFETCH: the next chunk's loads are in flight while a chunk is consumed (small batches).
template <bool PREFETCH>
__global__ void __launch_bounds__(kRHQ) k_route_pass(QueryArgs a, int l0, const uint32_t* __restrict__ order,
                                                     int32_t* __restrict__ cnt) {
    extern __shared__ __align__(16) float rt_smem[];
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const int d = a.d, ds = a.ds;
    const int nl = min(3, a.depth - l0);
    const int nn = (1 << nl) - 1;
    float* nvec = rt_smem;                                  // [7][ds]: the leader's subtree
    float* tile = rt_smem + (size_t)7 * ds + (size_t)warp * 32 * kRHP;
    const int64_t pb = blockIdx.x * (int64_t)kRHQ;
    const int vbase = (1 << l0) - 1;                        // first node of level l0
    const int v_lead = vbase + (l0 ? a.qleaf[order ? order[pb] : pb] : 0);
    auto node_of = [&](int v, int i) {                      // heap index of subtree entry i below v
        const int ll = i == 0 ? 0 : (i < 3 ? 1 : 2);
        return ((v + 1) << ll) - 1 + (i - ((1 << ll) - 1));
    };
    for (int e = threadIdx.x; e < nn * (ds >> 2); e += kRHQ) {
        const int i = e / (ds >> 2), c4 = e - i * (ds >> 2);
        const int nid = node_of(v_lead, i);
        const float* src = (a.ntype[nid] != 0 ? a.mu : a.dirs) + (size_t)nid * ds;
        reinterpret_cast<float4*>(nvec + (size_t)i * ds)[c4] = __ldg(reinterpret_cast<const float4*>(src) + c4);
    }
    __syncthreads();
    const int64_t p0 = pb + warp * 32;
    if (p0 >= a.nq) return;
    const int nrow = (int)min((int64_t)32, a.nq - p0);
    const bool act = lane < nrow;
    const int64_t q = act ? (order ? (int64_t)order[p0 + lane] : p0 + lane) : 0;
    const int v = act ? vbase + (l0 ? a.qleaf[q] : 0) : v_lead;
    const bool lead = __all_sync(BLSH_FULL, v == v_lead);
    const float* vec[7];
    bool mean[7];
    bool anymean = false;
#pragma unroll
    for (int i = 0; i < 7; ++i) {
        const bool use = i < nn;
        const int nid = use ? node_of(v, i) : 0;
        mean[i] = use && a.ntype[nid] != 0;
        vec[i] = lead ? nvec + (size_t)i * ds : ((mean[i] ? a.mu : a.dirs) + (size_t)nid * ds);
        anymean |= act && mean[i];
    }
    const bool generic = __any_sync(BLSH_FULL, anymean);
    auto qid = [&](int r) { return order ? (int64_t)order[p0 + r] : p0 + r; };
    float s[7];
#pragma unroll
    for (int i = 0; i < 7; ++i) s[i] = 0.0f;
    ChunkStager cst;
    if (PREFETCH) cst.load(a.Q, ds, qid, nrow, 0, lane);
    for (int j0 = 0; j0 < d; j0 += 32) {
        if (!PREFETCH) cst.load(a.Q, ds, qid, nrow, j0, lane);
        cst.store(tile, lane);
        __syncwarp();
        if (PREFETCH && j0 + 32 < d) cst.load(a.Q, ds, qid, nrow, j0 + 32, lane);
        const int jn = min(32, d - j0);
        const float* xr = tile + lane * kRHP;
        if (!generic && jn == 32) {   // hyperplane nodes only: s_i = fmaf(dir_ij, x_j, s_i)
#pragma unroll 2
            for (int jj = 0; jj < 32; jj += 4) {
                const float4 x = *reinterpret_cast<const float4*>(xr + jj);
#pragma unroll
                for (int i = 0; i < 7; ++i) {
                    if (i < nn) {
                        const float4 w = lead ? *reinterpret_cast<const float4*>(vec[i] + j0 + jj)
                                              : __ldg(reinterpret_cast<const float4*>(vec[i] + j0 + jj));
                        s[i] = __fmaf_rn(w.x, x.x, s[i]);
                        s[i] = __fmaf_rn(w.y, x.y, s[i]);
                        s[i] = __fmaf_rn(w.z, x.z, s[i]);
                        s[i] = __fmaf_rn(w.w, x.w, s[i]);
                    }
                }
            }
        } else {          // a mean-rule node somewhere (R4: s_i += (x_j - mu_ij)^2), or a ragged chunk
            for (int jj = 0; jj < jn; ++jj) {
                const float x = xr[jj];
#pragma unroll
                for (int i = 0; i < 7; ++i) {
                    if (i < nn) {
                        const float w = vec[i][j0 + jj];
                        const float e = __fsub_rn(x, w);
                        s[i] = mean[i] ? __fmaf_rn(e, e, s[i]) : __fmaf_rn(w, x, s[i]);
                    }
                }
            }
        }
        __syncwarp();
    }
    if (!act) return;
    int li = 0;
    for (int ll = 0; ll < nl; ++ll) {
        const int nid = node_of(v, li);
        float sl = s[0];
#pragma unroll
        for (int i = 1; i < 7; ++i) sl = i == li ? s[i] : sl;
        li = 2 * li + 1 + (sl > a.theta[nid] ? 1 : 0);
    }
    const int vn = ((v + 1) << nl) - 1 + (li - ((1 << nl) - 1));   // node reached (level l0 + nl)
    const int rel = vn - ((1 << (l0 + nl)) - 1);
    a.qleaf[q] = rel;
    atomicAdd(&cnt[rel], 1);
}

// exclusive scan of the G leaf counts into the scatter cursors (one block)
__global__ void __launch_bounds__(1024) k_leaf_scan(const int32_t* __restrict__ lcnt, int G, int32_t* __restrict__ lcur) {
    __shared__ int32_t wsum[32];
    const int per = (G + 1023) / 1024;
    const int lo = threadIdx.x * per, hi = min(G, lo + per);
    int32_t c = 0;
    for (int i = lo; i < hi; ++i) c += lcnt[i];
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    int32_t inc = c;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const int32_t y = __shfl_up_sync(BLSH_FULL, inc, o);
        if (lane >= o) inc += y;
    }
    if (lane == 31) wsum[w] = inc;
    __syncthreads();
    if (w == 0) {
        int32_t x = wsum[lane], xi = x;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const int32_t y = __shfl_up_sync(BLSH_FULL, xi, o);
            if (lane >= o) xi += y;
        }
        wsum[lane] = xi - x;
    }
    __syncthreads();
    int32_t run = wsum[w] + inc - c;
    for (int i = lo; i < hi; ++i) {
        lcur[i] = run;
        run += lcnt[i];
    }
}

__global__ void k_leaf_scatter(const int32_t* __restrict__ qleaf, int64_t nq, int32_t* __restrict__ lcur,
                               uint32_t* __restrict__ lperm) {
    const int64_t q = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (q < nq) lperm[atomicAdd(&lcur[qleaf[q]], 1)] = (uint32_t)q;
}

template <int MM>
__device__ __forceinline__ void hash_body(const QueryArgs& a, const uint32_t* __restrict__ lperm, float* smem) {
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const int64_t pb = blockIdx.x * (int64_t)kRHQ;
    const int d = a.d, ds = a.ds;
    float* As = smem;                                   // [MM][ds] of the block's first query's leaf
    float* tile = smem + (size_t)MM * ds + (size_t)warp * 32 * kRHP;
    const int g0 = a.qleaf[lperm[pb]];
    const float* Ag0 = a.A + (size_t)g0 * MM * d;
    for (int i = threadIdx.x; i < MM * d; i += kRHQ) {
        const int r = i / d, c = i - r * d;
        As[(size_t)r * ds + c] = __ldg(Ag0 + i);
    }
    __syncthreads();
    const int64_t p0 = pb + warp * 32;
    if (p0 >= a.nq) return;
    const int nrow = (int)min((int64_t)32, a.nq - p0);
    const bool act = lane < nrow;
    const int64_t q = act ? lperm[p0 + lane] : 0;
    const int g = act ? a.qleaf[q] : g0;
    const bool shared_a = __all_sync(BLSH_FULL, g == g0);
    const float* Ag = a.A + (size_t)g * MM * d;        // generic path: this lane's leaf, row pitch d
    auto qid = [&](int r) { return (int64_t)lperm[p0 + r]; };
    float s[MM];
#pragma unroll
    for (int i = 0; i < MM; ++i) s[i] = 0.0f;
    ChunkStager cst;
    cst.load(a.Q, ds, qid, nrow, 0, lane);
    for (int j0 = 0; j0 < d; j0 += 32) {
        cst.store(tile, lane);
        __syncwarp();
        if (j0 + 32 < d) cst.load(a.Q, ds, qid, nrow, j0 + 32, lane);   // in flight during this chunk
        const int jn = min(32, d - j0);
        const float* xr = tile + lane * kRHP;
        if (shared_a && jn == 32) {   // the block's leaf: broadcast 16-byte reads of A_g
#pragma unroll 1
            for (int jj = 0; jj < 32; jj += 4) {
                const float4 x = *reinterpret_cast<const float4*>(xr + jj);
#pragma unroll
                for (int i = 0; i < MM; ++i) {
                    const float4 w = *reinterpret_cast<const float4*>(As + (size_t)i * ds + j0 + jj);
                    s[i] = __fmaf_rn(w.x, x.x, s[i]);
                    s[i] = __fmaf_rn(w.y, x.y, s[i]);
                    s[i] = __fmaf_rn(w.z, x.z, s[i]);
                    s[i] = __fmaf_rn(w.w, x.w, s[i]);
                }
            }
        } else {
            for (int jj = 0; jj < jn; ++jj) {
                const float x = xr[jj];
                const int j = j0 + jj;
#pragma unroll
                for (int i = 0; i < MM; ++i)
                    s[i] = __fmaf_rn(g == g0 ? As[(size_t)i * ds + j] : __ldg(Ag + (size_t)i * d + j), x, s[i]);
            }
        }
        __syncwarp();
    }
    if (!act) return;
    const bool active = g >= a.leaf_lo && g < a.leaf_hi;
    const float W = a.Wl[g];
    float t[MM];
#pragma unroll
    for (int i = 0; i < MM; ++i) {
        t[i] = __fdiv_rn(__fadd_rn(s[i], a.bvec[g * MM + i]), W);
        a.qt[(size_t)q * MM + i] = t[i];
    }
    int32_t code[MM];
    const bool ok = quantise(t, MM, a.B, a.quantizer, code);
#pragma unroll
    for (int i = 0; i < MM; ++i) a.qcode[(size_t)q * MM + i] = code[i];
    bool fin = true;   // R30: a non-finite projection (NaN/Inf query) has no probes and no candidates
#pragma unroll
    for (int i = 0; i < MM; ++i) fin = fin && (__float_as_uint(t[i]) & 0x7F800000u) != 0x7F800000u;   // exponent bits
    a.qoor[q] = !fin ? 5 : (ok ? 0 : 1);
    a.qkey[q] = morton_key(code, MM, a.B);   // clamped home key (hierarchy uses it)
    if (!active) a.qoor[q] |= 2;
}

template <int MM>
__global__ void __launch_bounds__(kRHQ) k_hash(QueryArgs a, const uint32_t* __restrict__ lperm) {
    extern __shared__ __align__(16) float rh_smem[];
    hash_body<MM>(a, lperm, rh_smem);
}

// a2 of hash tables 1..L-1 in one launch (blockIdx.y = table - 1): the tables'
// blocks run together instead of one latency-bound launch per table.
template <int MM>
__global__ void __launch_bounds__(kRHQ) k_hash_tables(QueryArgs a, const __grid_constant__ HashTables ht) {
    extern __shared__ __align__(16) float rh_smem[];
    const int t = blockIdx.y;
    QueryArgs b = a;
    b.A = ht.A[t]; b.bvec = ht.b[t]; b.qt = ht.qt[t]; b.qcode = ht.qcode[t]; b.qoor = ht.qoor[t]; b.qkey = ht.qkey[t];
    hash_body<MM>(b, a.lperm, rh_smem);
}

// ---------------------------------------------------------------------------
// a3 + a4
// ---------------------------------------------------------------------------
__device__ __forceinline__ int64_t find_bucket(const Key128* __restrict__ ukey, int64_t lo, int64_t hi,
                                               const Key128& k) {
    const int64_t end = hi;
    // lower bound, 4-ary while the range is wide: the three pivot loads are
    // independent, so the dependent-load chain is half the binary one
    while (hi - lo > 3) {
        const int64_t n = hi - lo;
        const int64_t m1 = lo + (n >> 2), m2 = lo + (n >> 1), m3 = lo + ((3 * n) >> 2);
        const Key128 k1 = ukey[m1], k2 = ukey[m2], k3 = ukey[m3];
        if (key_lt(k3, k)) lo = m3 + 1;
        else if (key_lt(k2, k)) { lo = m2 + 1; hi = m3; }
        else if (key_lt(k1, k)) { lo = m1 + 1; hi = m2; }
        else hi = m1;
    }
    while (lo < hi) {
        const int64_t mid = (lo + hi) >> 1;
        const Key128 m = ukey[mid];
        if (key_lt(m, k)) lo = mid + 1;
        else hi = mid;
    }
    if (lo < end && key_eq(ukey[lo], k)) return lo;
    return -1;
}

constexpr int kPW = 4;          // warps per block in k_probe_lookup
constexpr int kMaxSel = 256;    // max probes (T <= 256)

constexpr int kFCap = 256;      // multiprobe frontier capacity (larger sets fall back to the pool)

struct ProbeSmem {
    uint32_t hist[256];
    unsigned long long sbits[kMaxSel];
    uint32_t sx[kMaxSel];
    uint32_t order[kMaxSel];
    uint32_t order2[16];        // recursive E8 probing: the selected second-ring vectors
    double fs[2][kFCap];        // frontier: partial scores
    uint32_t fe[2][kFCap];      // frontier: partial enc (base-3 digits delta_i + 1, i = 0 most significant)
};

__device__ __forceinline__ double ring2_score(const float* y, const int32_t* c2, uint32_t r) {
    int32_t p[8];
#pragma unroll
    for (int j = 0; j < 8; ++j) p[j] = c2[j] + (int32_t)g_e8_ring2[r][j];
    return e8_dist2(y, p);
}

// M = 16 (two E8 blocks, R28): candidate x moves block x / 240 by root x % 240;
// fp64 distance over all 16 coordinates (fma-accumulated, ascending j).
__device__ __forceinline__ double lat2_score(const float* y, const int32_t* c2, uint32_t x) {
    const uint32_t blk = x / 240u, r = x - blk * 240u;
    double s = 0.0;
#pragma unroll
    for (int j = 0; j < 16; ++j) {
        const int32_t c = c2[j] + ((uint32_t)(j >> 3) == blk ? (int32_t)c_e8_roots[r][j & 7] : 0);
        const double e = __dsub_rn((double)y[j], __dmul_rn(0.5, (double)c));
        s = __fma_rn(e, e, s);
    }
    return s;
}

__device__ __forceinline__ double lat_score(const float* y, const int32_t* c2, uint32_t r) {
    int32_t p[8];
#pragma unroll
    for (int j = 0; j < 8; ++j) p[j] = c2[j] + (int32_t)c_e8_roots[r][j];
    return e8_dist2(y, p);
}

// Select the R smallest (score, pool index) of a pool with an exact warp radix
// select over the fp64 score bits (scores >= 0: bit order == value order).
// Writes the selection sorted by (score, index) into sm.order[0..R).
// Pools of up to 32 * kSelCache entries (the common case: the pruning bound keeps
// a few dozen) score every entry once into registers (lane l, slot c holds pool
// index l + 32 c); larger pools re-score in every pass.
constexpr int kSelCache = 8;

template <bool CACHED, typename ScoreFn>
__device__ void warp_select_impl(ProbeSmem& sm, uint32_t P, uint32_t skip, int R, ScoreFn score) {
    const int lane = threadIdx.x & 31;
    unsigned long long sc[CACHED ? kSelCache : 1];
    // key of pool entry x = lane + 32 c (~0 = not in the pool)
    auto key = [&](int c, uint32_t x) -> unsigned long long {
        if (CACHED) return sc[c];
        return (x < P && x != skip) ? (unsigned long long)__double_as_longlong(score(x)) : ~0ull;
    };
    const int nslot = (int)((P + 31) / 32);
    if (CACHED) {
#pragma unroll
        for (int c = 0; c < kSelCache; ++c) {
            const uint32_t x = lane + 32u * c;
            sc[c] = (x < P && x != skip) ? (unsigned long long)__double_as_longlong(score(x)) : ~0ull;
        }
    }
    unsigned long long prefix = 0ull, mask = 0ull;
    // bits common to every key are skipped: start at the byte of the highest differing bit
    unsigned long long kmin = ~0ull, kmax = 0ull;
    int nvalid = 0;
#pragma unroll
    for (int c = 0; c < (CACHED ? kSelCache : 1); ++c) {
        for (int cc = c; cc < nslot; cc += (CACHED ? nslot : 1)) {
            const uint32_t x = lane + 32u * cc;
            const unsigned long long b = key(c, x);
            if (b != ~0ull) {
                kmin = b < kmin ? b : kmin;
                kmax = b > kmax ? b : kmax;
                ++nvalid;
            }
            if (CACHED) break;
        }
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) nvalid += __shfl_xor_sync(BLSH_FULL, nvalid, o);
    // a pool with fewer than R keys (only for non-finite scores, R30): select what there is and
    // mark the remaining slots invalid (0xFFFFFFFF: an empty probe)
    if (nvalid < R) {
        for (int e = nvalid + lane; e < R; e += 32) sm.order[e] = 0xFFFFFFFFu;
        R = nvalid;
        __syncwarp();
        if (R == 0) return;
    }
    int r = R - 1;
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        const unsigned long long a0 = __shfl_xor_sync(BLSH_FULL, kmin, o);
        const unsigned long long a1 = __shfl_xor_sync(BLSH_FULL, kmax, o);
        kmin = a0 < kmin ? a0 : kmin;
        kmax = a1 > kmax ? a1 : kmax;
    }
    int sh0 = -8;
    if (kmin != kmax) {
        const int hb = 63 - __clzll((long long)(kmin ^ kmax));
        sh0 = (hb / 8) * 8;
        mask = sh0 + 8 >= 64 ? 0ull : ~((1ull << (sh0 + 8)) - 1ull);
        prefix = kmin & mask;
    } else {
        mask = ~0ull;
        prefix = kmin;
    }
    for (int sh = sh0; sh >= 0; sh -= 8) {
        for (int i = lane; i < 256; i += 32) sm.hist[i] = 0;
        __syncwarp();
#pragma unroll
        for (int c = 0; c < (CACHED ? kSelCache : 1); ++c) {
            for (int cc = c; cc < nslot; cc += (CACHED ? nslot : 1)) {
                const unsigned long long b = key(c, lane + 32u * cc);
                if (b != ~0ull && (b & mask) == prefix) atomicAdd(&sm.hist[(b >> sh) & 255ull], 1u);
                if (CACHED) break;
            }
        }
        __syncwarp();
        uint32_t loc[8], tot = 0;
#pragma unroll
        for (int i = 0; i < 8; ++i) { loc[i] = sm.hist[lane * 8 + i]; tot += loc[i]; }
        uint32_t inc = tot;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const uint32_t y = __shfl_up_sync(BLSH_FULL, inc, o);
            if (lane >= o) inc += y;
        }
        const uint32_t ex = inc - tot;
        const bool mine = (uint32_t)r >= ex && (uint32_t)r < inc;
        const unsigned who = __ballot_sync(BLSH_FULL, mine);
        const int src = __ffs(who) - 1;
        int dg = 0, nr = 0;
        if (mine) {
            uint32_t c = ex;
#pragma unroll
            for (int i = 0; i < 8; ++i) {
                if ((uint32_t)r < c + loc[i]) { dg = lane * 8 + i; nr = r - (int)c; break; }
                c += loc[i];
            }
        }
        dg = __shfl_sync(BLSH_FULL, dg, src);
        r = __shfl_sync(BLSH_FULL, nr, src);
        const uint32_t binc = __shfl_sync(BLSH_FULL, sm.hist[dg], 0);
        prefix |= (unsigned long long)dg << sh;
        mask |= 255ull << sh;
        __syncwarp();
        if ((uint32_t)r + 1u == binc) break;   // the whole bin is taken: no finer digit needed
    }
    // take every key whose masked bits are < prefix, plus the first r+1 (ascending index)
    // of those equal to it (either all of them, or exact ties after the last digit)
    int cnt = 0, ties = 0;
#pragma unroll
    for (int c = 0; c < (CACHED ? kSelCache : 1); ++c) {
        for (int cc = c; cc < nslot; cc += (CACHED ? nslot : 1)) {
            const uint32_t x = lane + 32u * cc;
            const unsigned long long b = key(c, x);
            const unsigned long long bm = b == ~0ull ? ~0ull : (b & mask);
            const bool tie = b != ~0ull && bm == prefix;
            const unsigned tm = __ballot_sync(BLSH_FULL, tie);
            const int my_tie = ties + __popc(tm & lanemask_lt());
            ties += __popc(tm);
            const bool sel = (b != ~0ull && bm < prefix) || (tie && my_tie <= r);
            const unsigned smk = __ballot_sync(BLSH_FULL, sel);
            if (sel) {
                const int at = cnt + __popc(smk & lanemask_lt());
                sm.sbits[at] = b;
                sm.sx[at] = x;
            }
            cnt += __popc(smk);
            if (CACHED) break;
        }
    }
    __syncwarp();
    // sort the R selected entries by (score bits, index): R <= 32 by a register
    // bitonic network over the lanes (keys are distinct: x is unique), else
    // rank by counting
    if (R <= 32) {
        unsigned long long b = lane < R ? sm.sbits[lane] : ~0ull;
        uint32_t x = lane < R ? sm.sx[lane] : 0xFFFFFFFFu;
#pragma unroll
        for (int kk = 2; kk <= 32; kk <<= 1) {
#pragma unroll
            for (int j = kk >> 1; j > 0; j >>= 1) {
                const unsigned long long pb = __shfl_xor_sync(BLSH_FULL, b, j);
                const uint32_t px = __shfl_xor_sync(BLSH_FULL, x, j);
                const bool p_lt = pb < b || (pb == b && px < x);
                const bool m_lt = b < pb || (b == pb && x < px);
                const bool keep_min = ((lane & j) == 0) == ((lane & kk) == 0);
                if (keep_min ? p_lt : m_lt) { b = pb; x = px; }
            }
        }
        if (lane < R) sm.order[lane] = x;
        __syncwarp();
        return;
    }
    for (int e = lane; e < R; e += 32) {
        const unsigned long long b = sm.sbits[e];
        const uint32_t x = sm.sx[e];
        int rk = 0;
        for (int f = 0; f < R; ++f) {
            const unsigned long long bf = sm.sbits[f];
            rk += (bf < b || (bf == b && sm.sx[f] < x)) ? 1 : 0;
        }
        sm.order[rk] = x;
    }
    __syncwarp();
}

template <typename ScoreFn>
__device__ void warp_select(ProbeSmem& sm, uint32_t P, uint32_t skip, int R, ScoreFn score) {
    if (P <= 32u * kSelCache) warp_select_impl<true>(sm, P, skip, R, score);
    else warp_select_impl<false>(sm, P, skip, R, score);
}


#include "probe_kernel.cuh"

// ---------------------------------------------------------------------------
// tau = lower median of |A0| over the batch (single block radix select).
// ---------------------------------------------------------------------------
__global__ void __launch_bounds__(1024) k_median(const int64_t* __restrict__ base, int64_t nq, int64_t* __restrict__ tau) {
    __shared__ uint32_t h[256];
    __shared__ unsigned long long s_prefix;
    __shared__ int64_t s_rank;
    if (threadIdx.x == 0) { s_prefix = 0; s_rank = (nq - 1) / 2; }
    unsigned long long mask = 0ull;
    for (int sh = 56; sh >= 0; sh -= 8) {
        if (threadIdx.x < 256) h[threadIdx.x] = 0;
        __syncthreads();
        const unsigned long long pre = s_prefix;
        for (int64_t i = threadIdx.x; i < nq; i += blockDim.x) {
            const unsigned long long v = (unsigned long long)base[i];
            if ((v & mask) == pre) atomicAdd(&h[(v >> sh) & 255ull], 1u);
        }
        __syncthreads();
        if (threadIdx.x == 0) {
            int64_t r = s_rank, c = 0;
            for (int dg = 0; dg < 256; ++dg) {
                if (r < c + (int64_t)h[dg]) { s_prefix = pre | ((unsigned long long)dg << sh); s_rank = r - c; break; }
                c += h[dg];
            }
        }
        mask |= 255ull << sh;
        __syncthreads();
    }
    if (threadIdx.x == 0) *tau = nq > 0 ? (int64_t)s_prefix : 0;
}

__device__ __forceinline__ int64_t lower_key(const Key128* __restrict__ ukey, int64_t lo, int64_t hi, const Key128& k) {
    while (lo < hi) {
        const int64_t mid = (lo + hi) >> 1;
        if (key_lt(ukey[mid], k)) lo = mid + 1;
        else hi = mid;
    }
    return lo;
}
__device__ __forceinline__ int64_t upper_key(const Key128* __restrict__ ukey, int64_t lo, int64_t hi, const Key128& k) {
    while (lo < hi) {
        const int64_t mid = (lo + hi) >> 1;
        if (key_le(ukey[mid], k)) lo = mid + 1;
        else hi = mid;
    }
    return lo;
}

__global__ void k_widen(QueryArgs a, const int64_t* __restrict__ tau_p, int64_t min_cand) {
    const int64_t q = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (q >= a.nq) return;
    const int64_t tau = min_cand > 0 ? min_cand : *tau_p;
    if ((a.qoor[q] & 6) || a.base[q] >= tau) return;
    const int g = a.qleaf[q];
    const int64_t ulo = a.leaf_u[g], uhi = a.leaf_u[g + 1];
    const int BM = a.B * a.M;
    const Key128 k0 = a.qkey[q];
    int cb = 0;
    int64_t s = 0, e = 0;
    for (int l = 1;; ++l) {
        cb = min(l * a.hstep, BM);
        Key128 lo = k0, hi = k0;
        if (cb >= 128) { lo = Key128{0, 0}; hi = Key128{~0ull, ~0ull}; }
        else if (cb >= 64) {
            const unsigned long long mh = cb == 64 ? 0ull : ((1ull << (cb - 64)) - 1ull);
            lo = Key128{k0.hi & ~mh, 0ull};
            hi = Key128{lo.hi | mh, ~0ull};
        } else {
            const unsigned long long ml = (1ull << cb) - 1ull;
            lo = Key128{k0.hi, k0.lo & ~ml};
            hi = Key128{k0.hi, lo.lo | ml};
        }
        const int64_t ua = lower_key(a.ukey, ulo, uhi, lo);
        const int64_t ub = upper_key(a.ukey, ua, uhi, hi);
        s = ua < ub ? (int64_t)a.uoff[ua] : 0;
        e = ua < ub ? (int64_t)a.uoff[ub] : 0;
        if (e - s >= tau || cb == BM) break;
    }
    uint2* ivl = a.ivl + (size_t)q * (a.T + 1);
    int64_t c = a.base[q];
    for (int p = 0; p < a.T; ++p) {
        const uint2 iv = ivl[p];
        if (iv.y > iv.x && (int64_t)iv.x >= s && (int64_t)iv.y <= e) {
            c -= (int64_t)(iv.y - iv.x);
            ivl[p] = make_uint2(0, 0);
        }
    }
    ivl[a.T] = make_uint2((uint32_t)s, (uint32_t)e);
    a.cnt[q] = c + (e - s);
    if (a.level) a.level[q] = cb;
}

// P:132's shared-MSB climb (R32, hierarchy = 2), one thread per query: s* = the larger
// number of leading bits the clamped home key shares with the leaf's keys just before and
// after its insertion position; when s* < msb_min (default B*M: the home bucket is empty)
// the query also takes the leaf's buckets whose keys share those s* bits with it (one
// contiguous bucket range, containing the neighbour), with k_widen's containment rule.
__device__ __forceinline__ int shared_msb(const Key128& x, const Key128& y, int BM) {
    const unsigned long long h = x.hi ^ y.hi, l = x.lo ^ y.lo;
    const int len = h ? 128 - __clzll((long long)h) : (l ? 64 - __clzll((long long)l) : 0);
    return BM - len;
}

__global__ void k_msb_climb(QueryArgs a) {
    const int64_t q = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (q >= a.nq) return;
    if (a.qoor[q] & 6) return;
    const int g = a.qleaf[q];
    const int64_t ulo = a.leaf_u[g], uhi = a.leaf_u[g + 1];
    if (uhi <= ulo) return;
    const int BM = a.B * a.M;
    const Key128 k0 = a.qkey[q];
    const int64_t p0 = lower_key(a.ukey, ulo, uhi, k0);
    int sstar = 0;
    if (p0 > ulo) sstar = max(sstar, shared_msb(k0, a.ukey[p0 - 1], BM));
    if (p0 < uhi) sstar = max(sstar, shared_msb(k0, a.ukey[p0], BM));
    const int sig = a.msb_min > 0 ? a.msb_min : BM;
    if (sstar >= sig) return;
    const int cb = BM - sstar;
    Key128 lo = k0, hi = k0;
    if (cb >= 128) { lo = Key128{0, 0}; hi = Key128{~0ull, ~0ull}; }
    else if (cb >= 64) {
        const unsigned long long mh = cb == 64 ? 0ull : ((1ull << (cb - 64)) - 1ull);
        lo = Key128{k0.hi & ~mh, 0ull};
        hi = Key128{lo.hi | mh, ~0ull};
    } else {
        const unsigned long long ml = (1ull << cb) - 1ull;
        lo = Key128{k0.hi, k0.lo & ~ml};
        hi = Key128{k0.hi, lo.lo | ml};
    }
    const int64_t ua = lower_key(a.ukey, ulo, uhi, lo);
    const int64_t ub = upper_key(a.ukey, ua, uhi, hi);
    const int64_t s = ua < ub ? (int64_t)a.uoff[ua] : 0;
    const int64_t e = ua < ub ? (int64_t)a.uoff[ub] : 0;
    uint2* ivl = a.ivl + (size_t)q * (a.T + 1);
    int64_t c = a.base[q];
    for (int p = 0; p < a.T; ++p) {
        const uint2 iv = ivl[p];
        if (iv.y > iv.x && (int64_t)iv.x >= s && (int64_t)iv.y <= e) {
            c -= (int64_t)(iv.y - iv.x);
            ivl[p] = make_uint2(0, 0);
        }
    }
    ivl[a.T] = make_uint2((uint32_t)s, (uint32_t)e);
    a.cnt[q] = c + (e - s);
    if (a.level) a.level[q] = cb;
}

}  // namespace

void launch_msb_climb(const QueryArgs& a, cudaStream_t s) {
    k_msb_climb<<<(unsigned)((a.nq + 127) / 128), 128, 0, s>>>(a);
    BLSH_LAUNCH_CHECK();
}

void upload_e8_roots() {
    // __constant__ / __device__ tables are per device: track the upload per device, under a lock
    static std::mutex mu;
    static std::vector<bool> done_dev;
    int dev = 0;
    BLSH_CUDA(cudaGetDevice(&dev));
    std::lock_guard<std::mutex> lk(mu);
    if ((size_t)dev < done_dev.size() && done_dev[dev]) return;
    int8_t roots[240][8] = {};
    int r = 0;
    for (int i = 0; i < 8; ++i)
        for (int j = i + 1; j < 8; ++j)
            for (int si = 0; si < 2; ++si)
                for (int sj = 0; sj < 2; ++sj) {
                    roots[r][i] = si ? -2 : 2;
                    roots[r][j] = sj ? -2 : 2;
                    ++r;
                }
    for (int mask = 0; mask < 256; ++mask) {
        if (__builtin_popcount(mask) & 1) continue;
        for (int j = 0; j < 8; ++j) roots[r][j] = ((mask >> j) & 1) ? -1 : 1;
        ++r;
    }
    BLSH_CUDA(cudaMemcpyToSymbol(c_e8_roots, roots, sizeof(roots)));
    // the second ring (R26): r + r' of norm^2 4, 6, 8 (doubled 16, 24, 32), sorted by (norm^2, lexicographic)
    std::vector<std::array<int8_t, 8>> ring;
    ring.reserve(240 * 240);
    for (int i = 0; i < 240; ++i)
        for (int j = 0; j < 240; ++j) {
            std::array<int8_t, 8> v{};
            int n2 = 0;
            for (int t = 0; t < 8; ++t) {
                v[t] = (int8_t)(roots[i][t] + roots[j][t]);
                n2 += v[t] * v[t];
            }
            if (n2 >= 16) ring.push_back(v);
        }
    auto norm2 = [](const std::array<int8_t, 8>& v) {
        int n = 0;
        for (int t = 0; t < 8; ++t) n += v[t] * v[t];
        return n;
    };
    std::sort(ring.begin(), ring.end(), [&](const std::array<int8_t, 8>& x, const std::array<int8_t, 8>& y) {
        const int nx = norm2(x), ny = norm2(y);
        if (nx != ny) return nx < ny;
        return x < y;   // lexicographic on signed coordinates
    });
    ring.erase(std::unique(ring.begin(), ring.end()), ring.end());
    if (ring.size() != 9120) throw Error(BLSH_ERR_CUDA, "E8 second ring size");
    BLSH_CUDA(cudaMemcpyToSymbol(g_e8_ring2, ring.data(), ring.size() * 8));
    if ((size_t)dev >= done_dev.size()) done_dev.resize(dev + 1, false);
    done_dev[dev] = true;
}

constexpr int64_t kRoutePrefetchBelow = 16384;   // batches smaller than this fill < 1 wave of k_route
constexpr int64_t kRouteGroupFrom = 4096;        // regroup the queries between route passes from this batch size
// k_hash: A_g [M][ds] + one staged chunk per warp
static size_t hash_smem(const QueryArgs& a) {
    return ((size_t)a.M * a.ds + (size_t)kRHW * 32 * kRHP) * sizeof(float);
}

// a1: ceil(depth / 3) passes of k_route_pass, the queries regrouped by the node they reached
// between passes (k_leaf_scan / k_leaf_scatter over that level's nodes, into a.lperm); leaves in
// a.qleaf and the leaf histogram in a.lcnt[0, G) on return.  Returns the kernels launched.
static int launch_route(const QueryArgs& a, cudaStream_t s) {
    const unsigned grid = (unsigned)((a.nq + kRHQ - 1) / kRHQ);
    const size_t smem = ((size_t)7 * a.ds + (size_t)kRHW * 32 * kRHP) * sizeof(float);
    if (smem > 48 * 1024) {
        BLSH_CUDA(cudaFuncSetAttribute(k_route_pass<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
        BLSH_CUDA(cudaFuncSetAttribute(k_route_pass<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    }
    int launches = 0;
    const uint32_t* order = nullptr;
    for (int l0 = 0;; l0 += 3) {
        const int nl = std::max(0, std::min(3, a.depth - l0));
        const int nbins = 1 << (l0 + nl);
        BLSH_CUDA(cudaMemsetAsync(a.lcnt, 0, (size_t)nbins * sizeof(int32_t), s));
        if (a.nq < kRoutePrefetchBelow) k_route_pass<true><<<grid, kRHQ, smem, s>>>(a, l0, order, a.lcnt);
        else k_route_pass<false><<<grid, kRHQ, smem, s>>>(a, l0, order, a.lcnt);
        BLSH_LAUNCH_CHECK();
        ++launches;
        if (l0 + 3 >= a.depth) break;
        // small batches: no regrouping (two launches of latency for a few warps); their lanes
        // read their subtrees' vectors through L1
        if (a.nq < kRouteGroupFrom) continue;
        k_leaf_scan<<<1, 1024, 0, s>>>(a.lcnt, nbins, a.lcnt + a.G);
        BLSH_LAUNCH_CHECK();
        k_leaf_scatter<<<(unsigned)((a.nq + 255) / 256), 256, 0, s>>>(a.qleaf, a.nq, a.lcnt + a.G, a.lperm);
        BLSH_LAUNCH_CHECK();
        launches += 2;
        order = a.lperm;
    }
    return launches;
}

int launch_route_hash(const QueryArgs& a, cudaStream_t s) {
    if (a.nq == 0) return 0;
    const unsigned grid = (unsigned)((a.nq + kRHQ - 1) / kRHQ);
    const size_t smem_h = hash_smem(a);
    int32_t* lcnt = a.lcnt;
    int32_t* lcur = a.lcnt + a.G;
    int launches = launch_route(a, s);
    k_leaf_scan<<<1, 1024, 0, s>>>(lcnt, a.G, lcur);
    BLSH_LAUNCH_CHECK();
    k_leaf_scatter<<<(unsigned)((a.nq + 255) / 256), 256, 0, s>>>(a.qleaf, a.nq, lcur, a.lperm);
    BLSH_LAUNCH_CHECK();
#define BLSH_RH_CASE(MMV)                                                                                   \
    case MMV:                                                                                              \
        if (smem_h > 48 * 1024)                                                                            \
            BLSH_CUDA(cudaFuncSetAttribute(k_hash<MMV>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem_h)); \
        k_hash<MMV><<<grid, kRHQ, smem_h, s>>>(a, a.lperm);                                                 \
        break;
    switch (a.M) {
        BLSH_RH_CASE(1) BLSH_RH_CASE(2) BLSH_RH_CASE(3) BLSH_RH_CASE(4)
        BLSH_RH_CASE(5) BLSH_RH_CASE(6) BLSH_RH_CASE(7) BLSH_RH_CASE(8)
        BLSH_RH_CASE(9) BLSH_RH_CASE(10) BLSH_RH_CASE(11) BLSH_RH_CASE(12)
        BLSH_RH_CASE(13) BLSH_RH_CASE(14) BLSH_RH_CASE(15) BLSH_RH_CASE(16)
        default: throw Error(BLSH_ERR_INVALID, "M out of range");
    }
#undef BLSH_RH_CASE
    BLSH_LAUNCH_CHECK();
    return launches + 3;
}

// a1 alone over a batch, queries grouped by leaf (lperm), leaf counts in a.lcnt[0..G):
// the sharded path's first pass (run_query: a rank routes the whole batch, then works
// on the queries of its own leaves only).
int launch_route_group(const QueryArgs& a, cudaStream_t s) {
    if (a.nq == 0) return 0;
    int launches = launch_route(a, s);
    k_leaf_scan<<<1, 1024, 0, s>>>(a.lcnt, a.G, a.lcnt + a.G);
    BLSH_LAUNCH_CHECK();
    k_leaf_scatter<<<(unsigned)((a.nq + 255) / 256), 256, 0, s>>>(a.qleaf, a.nq, a.lcnt + a.G, a.lperm);
    BLSH_LAUNCH_CHECK();
    return launches + 2;
}

namespace {
// compact batch: row i = query idx[i] of the full batch (ds floats per row, 16-byte vectors)
__global__ void k_gather_rows(const float* __restrict__ Q, int ds, const uint32_t* __restrict__ idx, int64_t n,
                              float* __restrict__ out) {
    const int nv = ds >> 2;
    const int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (t >= n * nv) return;
    const int64_t i = t / nv;
    const int v = (int)(t - i * nv);
    reinterpret_cast<float4*>(out)[t] = __ldg(reinterpret_cast<const float4*>(Q + (size_t)idx[i] * ds) + v);
}
// full outputs: padding everywhere, then the compact rows at their queries
__global__ void k_shard_pad(int64_t nq, int k, int64_t* ids, float* d2, unsigned long long* pk, int64_t* nc) {
    const int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (t < nq * k) {
        if (ids) ids[t] = -1;
        if (d2) d2[t] = __int_as_float(0x7F800000);
        if (pk) pk[t] = 0x7F800000FFFFFFFFull;
    }
    if (nc && t < nq) nc[t] = 0;
}
__global__ void k_shard_scatter(const uint32_t* __restrict__ idx, int64_t n, int k, const int64_t* ids_c,
                                const float* d2_c, const unsigned long long* pk_c, const int64_t* nc_c, int64_t* ids,
                                float* d2, unsigned long long* pk, int64_t* nc) {
    const int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (t >= n * k) return;
    const int64_t i = t / k;
    const int j = (int)(t - i * k);
    const int64_t o = (int64_t)idx[i] * k + j;
    if (ids) ids[o] = ids_c[t];
    if (d2) d2[o] = d2_c[t];
    if (pk) pk[o] = pk_c[t];
    if (nc && j == 0) nc[idx[i]] = nc_c[i];
}
}  // namespace

void launch_gather_rows(const float* Q, int ds, const uint32_t* idx, int64_t n, float* out, cudaStream_t s) {
    if (n == 0) return;
    const int64_t tot = n * (ds >> 2);
    k_gather_rows<<<(unsigned)((tot + 255) / 256), 256, 0, s>>>(Q, ds, idx, n, out);
    BLSH_LAUNCH_CHECK();
}

void launch_shard_outputs(const uint32_t* idx, int64_t nq, int64_t n, int k, const int64_t* ids_c, const float* d2_c,
                          const unsigned long long* pk_c, const int64_t* nc_c, int64_t* ids, float* d2,
                          unsigned long long* pk, int64_t* nc, cudaStream_t s) {
    const int64_t tp = std::max<int64_t>(nq * k, nq);
    k_shard_pad<<<(unsigned)((tp + 255) / 256), 256, 0, s>>>(nq, k, ids, d2, pk, nc);
    BLSH_LAUNCH_CHECK();
    if (n > 0) {
        k_shard_scatter<<<(unsigned)((n * k + 255) / 256), 256, 0, s>>>(idx, n, k, ids_c, d2_c, pk_c, nc_c, ids, d2,
                                                                      pk, nc);
        BLSH_LAUNCH_CHECK();
    }
}

void launch_hash(const QueryArgs& a, cudaStream_t s) {
    if (a.nq == 0) return;
    const unsigned grid = (unsigned)((a.nq + kRHQ - 1) / kRHQ);
    const size_t smem_h = hash_smem(a);
#define BLSH_H_CASE(MMV)                                                                                    \
    case MMV:                                                                                              \
        if (smem_h > 48 * 1024)                                                                            \
            BLSH_CUDA(cudaFuncSetAttribute(k_hash<MMV>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem_h)); \
        k_hash<MMV><<<grid, kRHQ, smem_h, s>>>(a, a.lperm);                                                 \
        break;
    switch (a.M) {
        BLSH_H_CASE(1) BLSH_H_CASE(2) BLSH_H_CASE(3) BLSH_H_CASE(4)
        BLSH_H_CASE(5) BLSH_H_CASE(6) BLSH_H_CASE(7) BLSH_H_CASE(8)
        BLSH_H_CASE(9) BLSH_H_CASE(10) BLSH_H_CASE(11) BLSH_H_CASE(12)
        BLSH_H_CASE(13) BLSH_H_CASE(14) BLSH_H_CASE(15) BLSH_H_CASE(16)
        default: throw Error(BLSH_ERR_INVALID, "M out of range");
    }
#undef BLSH_H_CASE
    BLSH_LAUNCH_CHECK();
}

void launch_hash_tables(const QueryArgs& a, const HashTables& ht, cudaStream_t s) {
    if (a.nq == 0 || ht.n == 0) return;
    const dim3 grid((unsigned)((a.nq + kRHQ - 1) / kRHQ), (unsigned)ht.n);
    const size_t smem_h = hash_smem(a);
#define BLSH_HT_CASE(MMV)                                                                                     \
    case MMV:                                                                                                \
        if (smem_h > 48 * 1024)                                                                              \
            BLSH_CUDA(cudaFuncSetAttribute(k_hash_tables<MMV>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem_h)); \
        k_hash_tables<MMV><<<grid, kRHQ, smem_h, s>>>(a, ht);                                                 \
        break;
    switch (a.M) {
        BLSH_HT_CASE(1) BLSH_HT_CASE(2) BLSH_HT_CASE(3) BLSH_HT_CASE(4)
        BLSH_HT_CASE(5) BLSH_HT_CASE(6) BLSH_HT_CASE(7) BLSH_HT_CASE(8)
        BLSH_HT_CASE(9) BLSH_HT_CASE(10) BLSH_HT_CASE(11) BLSH_HT_CASE(12)
        BLSH_HT_CASE(13) BLSH_HT_CASE(14) BLSH_HT_CASE(15) BLSH_HT_CASE(16)
        default: throw Error(BLSH_ERR_INVALID, "M out of range");
    }
#undef BLSH_HT_CASE
    BLSH_LAUNCH_CHECK();
}

void launch_probe_lookup(const QueryArgs& a, cudaStream_t s) {
    if (a.T == 1 && a.probe != 3) {   // standard probing: thread per query
        k_lookup_home<<<(unsigned)((a.nq + 255) / 256), 256, 0, s>>>(a);
        BLSH_LAUNCH_CHECK();
        return;
    }
    k_probe_lookup<<<(unsigned)((a.nq + kPW - 1) / kPW), kPW * 32, 0, s>>>(a);
    BLSH_LAUNCH_CHECK();
}

void launch_median(const int64_t* base, int64_t nq, int64_t* tau, cudaStream_t s) {
    k_median<<<1, 1024, 0, s>>>(base, nq, tau);
    BLSH_LAUNCH_CHECK();
}

void launch_widen(const QueryArgs& a, const int64_t* tau, int64_t min_cand, cudaStream_t s) {
    k_widen<<<(unsigned)((a.nq + 127) / 128), 128, 0, s>>>(a, tau, min_cand);
    BLSH_LAUNCH_CHECK();
}

}  // namespace blsh
