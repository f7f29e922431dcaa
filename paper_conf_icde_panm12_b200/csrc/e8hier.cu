// e8hier.cu -- the E8 code hierarchy (Eq. 10; reading R27).
//
// "There is no compact representation of E8 LSH hierarchy similar to the
// Morton curve ... We implement the E8 hierarchy as a linear array along with
// an index hierarchy".  Here: for every level j = 1..J the buckets of
// the (primary) table, re-keyed by their level-j code a_j(u) = parent^j(c_u),
// parent(c) = DECODE(c / 2) (doubled coordinates: DECODE(c2 / 4)), sorted by
// (leaf, Morton(a_j), u) with the running row count -- a node of level j is one
// equal-key run of that array (binary search), its size one subtraction.  The
// table rows themselves stay in the level-0 (Morton) order.
//
// Build: J rounds of (parent of every bucket code, key, LSD radix sort of
// (leaf, key, u), bucket sizes in sorted order, scan); a leaf's root level m_g
// is the first level at which its first and last entries share a key.
// Query (k_e8_widen): thread per query, the query's chain a_j(q) computed on
// the fly; the first level j <= m_g whose node contains a_j(q) with >= tau rows
// (else the whole leaf).  Candidates = A0 u node, deduplicated by the bitmap
// union (tables.cu) and streamed by the list-mode warp short-list.
#include "hashcore.cuh"
#include "internal.cuh"
#include "query_kernels.cuh"

namespace blsh {

namespace {

__device__ __forceinline__ void morton_decode(const Key128& k, int M, int B, int32_t* code) {
    const int off = 1 << (B - 1);
    for (int i = 0; i < M; ++i) {
        uint32_t u = 0;
        const int base = M - 1 - i;
        for (int p = 0; p < B; ++p) {
            const int pos = p * M + base;
            const unsigned long long bit = pos < 64 ? (k.lo >> pos) & 1ull : (k.hi >> (pos - 64)) & 1ull;
            u |= (uint32_t)bit << p;
        }
        code[i] = (int32_t)u - off;
    }
}

__device__ __forceinline__ void e8_parent(const int32_t* c2, int32_t* out) {
    float y[8];
#pragma unroll
    for (int i = 0; i < 8; ++i) y[i] = __fmul_rn((float)c2[i], 0.25f);
    e8_decode(y, out);
}

// level 0 codes of every bucket
__global__ void k_bucket_codes(const Key128* __restrict__ ukey, int64_t nu, int M, int B, int32_t* __restrict__ codes) {
    for (int64_t u = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; u < nu; u += (int64_t)gridDim.x * blockDim.x)
        morton_decode(ukey[u], M, B, codes + (size_t)M * u);
}

// one level up: codes <- parent(codes); sort entries (leaf, key, u)
__global__ void k_parent_level(int32_t* __restrict__ codes, const int32_t* __restrict__ uleaf, int64_t nu, int M, int B,
                               unsigned long long* __restrict__ hi, unsigned long long* __restrict__ lo,
                               uint32_t* __restrict__ leaf, uint32_t* __restrict__ id) {
    for (int64_t u = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; u < nu; u += (int64_t)gridDim.x * blockDim.x) {
        int32_t c[16], p[16];
        for (int i = 0; i < M; ++i) c[i] = codes[(size_t)M * u + i];
        for (int blk = 0; blk < M / 8; ++blk) e8_parent(c + 8 * blk, p + 8 * blk);   // per block (R28)
        for (int i = 0; i < M; ++i) codes[(size_t)M * u + i] = p[i];
        const Key128 k = morton_key(p, M, B);
        hi[u] = k.hi;
        lo[u] = k.lo;
        leaf[u] = (uint32_t)uleaf[u];
        id[u] = (uint32_t)u;
    }
}

__global__ void k_level_store(const unsigned long long* __restrict__ hi, const unsigned long long* __restrict__ lo,
                              const uint32_t* __restrict__ id, const uint32_t* __restrict__ uoff, int64_t nu,
                              Key128* __restrict__ key, uint32_t* __restrict__ bu, int64_t* __restrict__ sz) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < nu; i += (int64_t)gridDim.x * blockDim.x) {
        const uint32_t u = id[i];
        key[i] = Key128{hi[i], lo[i]};
        bu[i] = u;
        sz[i] = (int64_t)uoff[u + 1] - (int64_t)uoff[u];
    }
}

__device__ __forceinline__ int64_t lower_k(const Key128* __restrict__ a, int64_t lo, int64_t hi, const Key128& k) {
    while (lo < hi) {
        const int64_t mid = (lo + hi) >> 1;
        if (key_lt(a[mid], k)) lo = mid + 1;
        else hi = mid;
    }
    return lo;
}
__device__ __forceinline__ int64_t upper_k(const Key128* __restrict__ a, int64_t lo, int64_t hi, const Key128& k) {
    while (lo < hi) {
        const int64_t mid = (lo + hi) >> 1;
        if (key_lt(k, a[mid])) hi = mid;
        else lo = mid + 1;
    }
    return lo;
}

__global__ void k_e8_widen(E8WidenArgs w, const int64_t* __restrict__ tau_p, int64_t min_cand) {
    const int64_t q = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (q >= w.nq) return;
    const int64_t tau = min_cand > 0 ? min_cand : *tau_p;
    w.hlevel[q] = 0;
    w.hrows[q] = 0;
    w.hs[q] = 0;
    w.he[q] = 0;
    if ((w.qoor[q] & 6) || w.base[q] >= tau) return;
    const int g = w.qleaf[q];
    const int64_t u0 = w.leaf_u[g], u1 = w.leaf_u[g + 1];
    const int M = w.M;
    int32_t c[16], p[16];
    for (int i = 0; i < M; ++i) c[i] = w.qcode[(size_t)M * q + i];
    int level = kE8Levels + 1;
    int64_t s = 0, e = 0, rows = 0;
    for (int j = 0; j <= kE8Levels && u1 > u0; ++j) {
        const Key128 k = morton_key(c, M, w.B);
        const Key128* K = j == 0 ? w.ukey : w.lv_key[j];
        const int64_t a = lower_k(K, u0, u1, k);
        const int64_t b = upper_k(K, a, u1, k);
        if (b > a) {
            const int64_t r = j == 0 ? (int64_t)w.uoff[b] - (int64_t)w.uoff[a] : w.lv_cum[j][b] - w.lv_cum[j][a];
            if (r >= tau) { level = j; s = a; e = b; rows = r; break; }
        }
        if (j >= w.root[g]) break;                 // root: every bucket of the leaf shares a_j
        for (int blk = 0; blk < M / 8; ++blk) e8_parent(c + 8 * blk, p + 8 * blk);
        for (int i = 0; i < M; ++i) c[i] = p[i];
    }
    if (level > kE8Levels) {                       // the whole leaf
        s = u0;
        e = u1;
        rows = (int64_t)w.uoff[u1] - (int64_t)w.uoff[u0];
    }
    w.hlevel[q] = level;
    w.hs[q] = s;
    w.he[q] = e;
    w.hrows[q] = rows;
}

}  // namespace

void build_e8_hierarchy(blsh_index& ix, cudaStream_t s) {
    const int64_t nu = ix.nu;
    ix.e8_levels = 0;
    ix.e8_root_h.assign(ix.G, 0);
    if (nu == 0) {
        ix.e8_root.alloc(ix.G * sizeof(int32_t));
        BLSH_CUDA(cudaMemsetAsync(ix.e8_root.p, 0, ix.G * sizeof(int32_t), s));
        return;
    }
    DevBuf codes;
    codes.alloc((size_t)nu * ix.M * sizeof(int32_t));
    k_bucket_codes<<<592, 256, 0, s>>>(ix.ukey.as<Key128>(), nu, ix.M, ix.B, codes.as<int32_t>());
    BLSH_LAUNCH_CHECK();
    SortBufs sb;
    for (int i = 0; i < 2; ++i) {
        sb.hi[i].alloc((size_t)nu * 8);
        sb.lo[i].alloc((size_t)nu * 8);
        sb.leaf[i].alloc((size_t)nu * 4);
        sb.id[i].alloc((size_t)nu * 4);
    }
    // root level per leaf: level 0 first (the table's own keys)
    std::vector<int64_t> lu = ix.leaf_u_h;
    std::vector<int32_t>& root = ix.e8_root_h;
    std::vector<Key128> kf(1), kl(1);
    auto leaf_same = [&](const Key128* keys, int g) {
        if (lu[g + 1] - lu[g] <= 1) return true;
        BLSH_CUDA(cudaMemcpy(kf.data(), keys + lu[g], sizeof(Key128), cudaMemcpyDeviceToHost));
        BLSH_CUDA(cudaMemcpy(kl.data(), keys + lu[g + 1] - 1, sizeof(Key128), cudaMemcpyDeviceToHost));
        return kf[0].hi == kl[0].hi && kf[0].lo == kl[0].lo;
    };
    std::vector<bool> done(ix.G, false);
    int open = 0;
    for (int g = ix.leaf_lo; g < ix.leaf_hi; ++g) {
        if (leaf_same(ix.ukey.as<Key128>(), g)) { done[g] = true; root[g] = 0; }
        else { root[g] = kE8Levels; ++open; }
    }
    ix.e8_key.clear();
    ix.e8_bu.clear();
    ix.e8_cum.clear();
    ix.e8_key.emplace_back();   // level 0 = the table itself (placeholders)
    ix.e8_bu.emplace_back();
    ix.e8_cum.emplace_back();
    ScanTemp scan;
    int passes = 0;
    for (int j = 1; j <= kE8Levels && open > 0; ++j) {
        k_parent_level<<<592, 256, 0, s>>>(codes.as<int32_t>(), ix.uleaf.as<int32_t>(), nu, ix.M, ix.B,
                                           sb.hi[0].as<unsigned long long>(), sb.lo[0].as<unsigned long long>(),
                                           sb.leaf[0].as<uint32_t>(), sb.id[0].as<uint32_t>());
        BLSH_LAUNCH_CHECK();
        const int cur = radix_sort_entries(sb, nu, s, &passes);
        auto K = std::make_unique<DevBuf>(), U = std::make_unique<DevBuf>(), C = std::make_unique<DevBuf>();
        K->alloc((size_t)nu * sizeof(Key128));
        U->alloc((size_t)nu * sizeof(uint32_t));
        C->alloc((size_t)(nu + 1) * sizeof(int64_t));
        DevBuf sz;
        sz.alloc((size_t)nu * sizeof(int64_t));
        k_level_store<<<592, 256, 0, s>>>(sb.hi[cur].as<unsigned long long>(), sb.lo[cur].as<unsigned long long>(),
                                          sb.id[cur].as<uint32_t>(), ix.uoff.as<uint32_t>(), nu, K->as<Key128>(),
                                          U->as<uint32_t>(), sz.as<int64_t>());
        BLSH_LAUNCH_CHECK();
        scan_exclusive_i64(sz.as<int64_t>(), C->as<int64_t>(), nu, scan, s);
        BLSH_CUDA(cudaStreamSynchronize(s));
        for (int g = ix.leaf_lo; g < ix.leaf_hi; ++g)
            if (!done[g] && leaf_same(K->as<Key128>(), g)) { done[g] = true; root[g] = j; --open; }
        ix.e8_key.push_back(std::move(K));
        ix.e8_bu.push_back(std::move(U));
        ix.e8_cum.push_back(std::move(C));
        ix.e8_levels = j;
    }
    ix.e8_root.alloc(ix.G * sizeof(int32_t));
    BLSH_CUDA(cudaMemcpyAsync(ix.e8_root.p, root.data(), ix.G * sizeof(int32_t), cudaMemcpyHostToDevice, s));
    std::vector<const Key128*> kp(kE8Levels + 1, nullptr);
    std::vector<const uint32_t*> bp(kE8Levels + 1, nullptr);
    std::vector<const int64_t*> cp(kE8Levels + 1, nullptr);
    for (int j = 1; j <= ix.e8_levels; ++j) {
        kp[j] = ix.e8_key[j]->as<Key128>();
        bp[j] = ix.e8_bu[j]->as<uint32_t>();
        cp[j] = ix.e8_cum[j]->as<int64_t>();
    }
    ix.e8_ptrs.alloc((size_t)3 * (kE8Levels + 1) * sizeof(void*));
    char* base = ix.e8_ptrs.as<char>();
    BLSH_CUDA(cudaMemcpyAsync(base, kp.data(), (kE8Levels + 1) * sizeof(void*), cudaMemcpyHostToDevice, s));
    BLSH_CUDA(cudaMemcpyAsync(base + (kE8Levels + 1) * sizeof(void*), bp.data(), (kE8Levels + 1) * sizeof(void*),
                              cudaMemcpyHostToDevice, s));
    BLSH_CUDA(cudaMemcpyAsync(base + 2 * (kE8Levels + 1) * sizeof(void*), cp.data(), (kE8Levels + 1) * sizeof(void*),
                              cudaMemcpyHostToDevice, s));
    BLSH_CUDA(cudaStreamSynchronize(s));
}

void launch_e8_widen(const E8WidenArgs& w, const int64_t* tau, int64_t min_cand, cudaStream_t s) {
    if (w.nq == 0) return;
    k_e8_widen<<<(unsigned)((w.nq + 127) / 128), 128, 0, s>>>(w, tau, min_cand);
    BLSH_LAUNCH_CHECK();
}

}  // namespace blsh
