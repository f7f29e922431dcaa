// build.cu -- b3 (hash every owned data point with its leaf's parameters,
// P:41 Eq. 2 / P:142 Eq. 6, Morton key P:130) and b4 (buckets as runs of the
// sorted bi-level code, plus the rows of X permuted into table order so
// every bucket and every Morton-prefix range is one contiguous slab of HBM).
#include <algorithm>

#include "hashcore.cuh"
#include "internal.cuh"

namespace blsh {

namespace {

constexpr int kTR = 256;

struct HTile {
    int32_t leaf;
    int32_t len;
    int64_t start;   // position in `order`
};

// One lane per row, 32 rows per warp, a tile of <= 256 rows of one leaf per block: the
// leaf's a_i in shared memory (pitch ds, broadcast 16-byte reads), the rows streamed as
// 32-column chunks staged by coalesced 16-byte loads (ChunkStager); M canonical fp32
// chains per lane (R1), then t_i = (dot + b_i) / W, quantise, Morton key.
template <int MM>
__global__ void __launch_bounds__(kTR) k_hash_rows(const float* __restrict__ Xs, int ds, int d,
                                                   const uint32_t* __restrict__ order,
                                                   const HTile* __restrict__ tiles, int64_t pos_lo,
                                                   const float* __restrict__ A, const float* __restrict__ bvec,
                                                   const float* __restrict__ Wl, int B, int quantizer,
                                                   unsigned long long* __restrict__ key_hi,
                                                   unsigned long long* __restrict__ key_lo,
                                                   uint32_t* __restrict__ leaf_o, uint32_t* __restrict__ id_o,
                                                   int32_t* __restrict__ code_out, int* __restrict__ bad) {
    extern __shared__ __align__(16) float hsm[];
    float* as_ = hsm;                                               // [MM][ds]
    float* tile = hsm + (size_t)MM * ds + (size_t)(threadIdx.x >> 5) * 32 * kRowPitch;
    const HTile t = tiles[blockIdx.x];
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const float* Ag = A + (size_t)t.leaf * MM * d;
    for (int i = threadIdx.x; i < MM * d; i += kTR) {
        const int ii = i / d, jj = i - ii * d;
        as_[(size_t)ii * ds + jj] = __ldg(Ag + i);
    }
    __syncthreads();
    const int r0 = warp * 32;
    if (r0 >= t.len) return;
    const int nrow = min(32, t.len - r0);
    const uint32_t* rid = order + t.start + r0;
    auto qid = [&](int r) { return (int64_t)rid[r]; };
    float s[MM];
#pragma unroll
    for (int i = 0; i < MM; ++i) s[i] = 0.0f;
    ChunkStager cst;
    cst.load(Xs, ds, qid, nrow, 0, lane);
    for (int j0 = 0; j0 < d; j0 += 32) {
        cst.store(tile, lane);
        __syncwarp();
        if (j0 + 32 < d) cst.load(Xs, ds, qid, nrow, j0 + 32, lane);   // in flight during this chunk
        const int jn = min(32, d - j0);
        const float* xr = tile + lane * kRowPitch;
        if (jn == 32) {
#pragma unroll 2
            for (int jj = 0; jj < 32; jj += 4) {
                const float4 x = *reinterpret_cast<const float4*>(xr + jj);
#pragma unroll
                for (int i = 0; i < MM; ++i) {
                    const float4 w = *reinterpret_cast<const float4*>(as_ + (size_t)i * ds + j0 + jj);
                    s[i] = __fmaf_rn(w.x, x.x, s[i]);
                    s[i] = __fmaf_rn(w.y, x.y, s[i]);
                    s[i] = __fmaf_rn(w.z, x.z, s[i]);
                    s[i] = __fmaf_rn(w.w, x.w, s[i]);
                }
            }
        } else {
            for (int jj = 0; jj < jn; ++jj) {
                const float x = xr[jj];
#pragma unroll
                for (int i = 0; i < MM; ++i) s[i] = __fmaf_rn(as_[(size_t)i * ds + j0 + jj], x, s[i]);
            }
        }
        __syncwarp();
    }
    if (lane >= nrow) return;
    const int r = r0 + lane;
    const float W = Wl[t.leaf];
    float tv[MM];
#pragma unroll
    for (int i = 0; i < MM; ++i) tv[i] = __fdiv_rn(__fadd_rn(s[i], bvec[t.leaf * MM + i]), W);
    int32_t code[MM];
    const bool ok = quantise(tv, MM, B, quantizer, code);
    if (!ok) atomicOr(bad, 1);
    const Key128 k = morton_key(code, MM, B);
    const int64_t o = t.start + r - pos_lo;
    const uint32_t id = rid[lane];
    key_hi[o] = k.hi;
    key_lo[o] = k.lo;
    leaf_o[o] = (uint32_t)t.leaf;
    id_o[o] = id;
    if (code_out) {
#pragma unroll
        for (int i = 0; i < MM; ++i) code_out[(size_t)id * MM + i] = code[i];
    }
}

__global__ void k_flags(const unsigned long long* __restrict__ hi, const unsigned long long* __restrict__ lo,
                        const uint32_t* __restrict__ leaf, int64_t n, uint8_t* __restrict__ f) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        f[i] = (i == 0 || hi[i] != hi[i - 1] || lo[i] != lo[i - 1] || leaf[i] != leaf[i - 1]) ? 1 : 0;
}

__global__ void k_unique(const unsigned long long* __restrict__ hi, const unsigned long long* __restrict__ lo,
                         const uint32_t* __restrict__ leaf, const uint32_t* __restrict__ id,
                         const uint8_t* __restrict__ f, const int64_t* __restrict__ U, int64_t n,
                         Key128* __restrict__ ukey, int32_t* __restrict__ uleaf, uint32_t* __restrict__ uoff,
                         uint32_t* __restrict__ perm) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
        perm[i] = id[i];
        if (f[i]) {
            const int64_t u = U[i];
            ukey[u] = Key128{hi[i], lo[i]};
            uleaf[u] = (int32_t)leaf[i];
            uoff[u] = (uint32_t)i;
        }
        if (i == n - 1) uoff[U[n]] = (uint32_t)n;
    }
}

__global__ void k_leaf_u(const int32_t* __restrict__ uleaf, int64_t nu, int G, int64_t* __restrict__ leaf_u) {
    const int g = blockIdx.x * blockDim.x + threadIdx.x;
    if (g > G) return;
    int64_t lo = 0, hi = nu;   // first u with uleaf[u] >= g
    while (lo < hi) {
        const int64_t mid = (lo + hi) >> 1;
        if (uleaf[mid] < g) lo = mid + 1;
        else hi = mid;
    }
    leaf_u[g] = lo;
}

// X_perm[pos] = X[perm[pos]]: one warp per row, 16-byte vectors.
__global__ void k_permute_rows(const float* __restrict__ Xs, int ds, const uint32_t* __restrict__ perm,
                               int64_t n, float* __restrict__ Xp) {
    const int lane = threadIdx.x & 31;
    const int64_t warps = (int64_t)gridDim.x * (blockDim.x >> 5);
    const int nv = ds >> 2;
    for (int64_t row = blockIdx.x * (int64_t)(blockDim.x >> 5) + (threadIdx.x >> 5); row < n; row += warps) {
        const float4* src = reinterpret_cast<const float4*>(Xs + (size_t)perm[row] * ds);
        float4* dst = reinterpret_cast<float4*>(Xp + (size_t)row * ds);
        for (int v = lane; v < nv; v += 32) dst[v] = src[v];
    }
}

__global__ void k_invert(const uint32_t* __restrict__ perm, int64_t n, uint32_t* __restrict__ inv) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        inv[perm[i]] = (uint32_t)i;
}

__global__ void k_map_pos(const uint32_t* __restrict__ perm_l, const uint32_t* __restrict__ inv0, int64_t n,
                          uint32_t* __restrict__ pos) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        pos[i] = inv0[perm_l[i]];
}

}  // namespace

void invert_perm(const uint32_t* perm, int64_t n_owned, uint32_t* inv, cudaStream_t s) {
    if (n_owned == 0) return;
    k_invert<<<592, 256, 0, s>>>(perm, n_owned, inv);
    BLSH_LAUNCH_CHECK();
}

void build_extra_table(const blsh_index& ix, ExtraTable& t, const unsigned long long* key_hi,
                       const unsigned long long* key_lo, const uint32_t* leaf, const uint32_t* id,
                       const uint32_t* inv0, int64_t n_owned, ScanTemp& scan, cudaStream_t s) {
    const int64_t n = n_owned;
    DevBuf flags, U;
    flags.alloc(std::max<int64_t>(n, 1));
    U.alloc((std::max<int64_t>(n, 1) + 1) * sizeof(int64_t));
    t.perm.alloc(std::max<int64_t>(n, 1) * sizeof(uint32_t));
    t.pos.alloc(std::max<int64_t>(n, 1) * sizeof(uint32_t));
    int64_t nu = 0;
    if (n > 0) {
        k_flags<<<592, 256, 0, s>>>(key_hi, key_lo, leaf, n, flags.as<uint8_t>());
        BLSH_LAUNCH_CHECK();
        scan_exclusive_u8(flags.as<uint8_t>(), U.as<int64_t>(), n, scan, s);
        BLSH_CUDA(cudaMemcpyAsync(&nu, U.as<int64_t>() + n, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
        BLSH_CUDA(cudaStreamSynchronize(s));
    }
    t.nu = nu;
    t.ukey.alloc(std::max<int64_t>(nu, 1) * sizeof(Key128));
    t.uleaf.alloc(std::max<int64_t>(nu, 1) * sizeof(int32_t));
    t.uoff.alloc((std::max<int64_t>(nu, 1) + 1) * sizeof(uint32_t));
    BLSH_CUDA(cudaMemsetAsync(t.uoff.p, 0, sizeof(uint32_t), s));
    if (n > 0) {
        k_unique<<<592, 256, 0, s>>>(key_hi, key_lo, leaf, id, flags.as<uint8_t>(), U.as<int64_t>(), n,
                                     t.ukey.as<Key128>(), t.uleaf.as<int32_t>(), t.uoff.as<uint32_t>(),
                                     t.perm.as<uint32_t>());
        BLSH_LAUNCH_CHECK();
        k_map_pos<<<592, 256, 0, s>>>(t.perm.as<uint32_t>(), inv0, n, t.pos.as<uint32_t>());
        BLSH_LAUNCH_CHECK();
    }
    t.leaf_u.alloc((ix.G + 1) * sizeof(int64_t));
    k_leaf_u<<<(ix.G + 1 + 127) / 128, 128, 0, s>>>(t.uleaf.as<int32_t>(), nu, ix.G, t.leaf_u.as<int64_t>());
    BLSH_LAUNCH_CHECK();
    t.leaf_u_h.assign(ix.G + 1, 0);
    BLSH_CUDA(cudaMemcpyAsync(t.leaf_u_h.data(), t.leaf_u.p, (ix.G + 1) * sizeof(int64_t), cudaMemcpyDeviceToHost, s));
    BLSH_CUDA(cudaStreamSynchronize(s));
}

bool hash_points(const blsh_index& ix, const float* Xs, const uint32_t* order, const std::vector<int64_t>& seg,
                 int64_t pos_lo, int64_t pos_hi, unsigned long long* key_hi, unsigned long long* key_lo,
                 uint32_t* leaf, uint32_t* id, int32_t* code_out, cudaStream_t s, const float* A,
                 const float* b) {
    if (!A) A = ix.A.as<float>();
    if (!b) b = ix.b.as<float>();
    std::vector<HTile> tiles;
    for (int g = ix.leaf_lo; g < ix.leaf_hi; ++g)
        for (int64_t p = seg[g]; p < seg[g + 1]; p += kTR)
            tiles.push_back(HTile{g, (int32_t)std::min<int64_t>(kTR, seg[g + 1] - p), p});
    if (tiles.empty()) return true;
    DevBuf tiles_d, bad_d;
    tiles_d.alloc(tiles.size() * sizeof(HTile));
    BLSH_CUDA(cudaMemcpyAsync(tiles_d.p, tiles.data(), tiles.size() * sizeof(HTile), cudaMemcpyHostToDevice, s));
    bad_d.alloc(sizeof(int));
    BLSH_CUDA(cudaMemsetAsync(bad_d.p, 0, sizeof(int), s));
    const unsigned nt = (unsigned)tiles.size();
    const size_t hsmem = ((size_t)ix.M * ix.ds + (size_t)(kTR / 32) * 32 * kRowPitch) * sizeof(float);
#define BLSH_HASH_CASE(MMV)                                                                                    \
    case MMV:                                                                                                  \
        BLSH_CUDA(cudaFuncSetAttribute(k_hash_rows<MMV>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)hsmem)); \
        k_hash_rows<MMV><<<nt, kTR, hsmem, s>>>(Xs, ix.ds, ix.d, order, tiles_d.as<HTile>(), pos_lo,              \
                                            A, b, ix.W.as<float>(), ix.B,                                     \
                                            ix.quantizer, key_hi, key_lo, leaf, id, code_out, bad_d.as<int>()); \
        break;
    switch (ix.M) {
        BLSH_HASH_CASE(1) BLSH_HASH_CASE(2) BLSH_HASH_CASE(3) BLSH_HASH_CASE(4)
        BLSH_HASH_CASE(5) BLSH_HASH_CASE(6) BLSH_HASH_CASE(7) BLSH_HASH_CASE(8)
        BLSH_HASH_CASE(9) BLSH_HASH_CASE(10) BLSH_HASH_CASE(11) BLSH_HASH_CASE(12)
        BLSH_HASH_CASE(13) BLSH_HASH_CASE(14) BLSH_HASH_CASE(15) BLSH_HASH_CASE(16)
        default: throw Error(BLSH_ERR_INVALID, "M out of range");
    }
#undef BLSH_HASH_CASE
    BLSH_LAUNCH_CHECK();
    int bad = 0;
    BLSH_CUDA(cudaMemcpyAsync(&bad, bad_d.p, sizeof(int), cudaMemcpyDeviceToHost, s));
    BLSH_CUDA(cudaStreamSynchronize(s));
    (void)pos_hi;
    return bad == 0;
}

void build_table(blsh_index& ix, const float* Xs, const unsigned long long* key_hi, const unsigned long long* key_lo,
                 const uint32_t* leaf, const uint32_t* id, int64_t n_owned, ScanTemp& scan, cudaStream_t s) {
    const int64_t n = n_owned;
    DevBuf flags, U;
    flags.alloc(std::max<int64_t>(n, 1));
    U.alloc((std::max<int64_t>(n, 1) + 1) * sizeof(int64_t));
    ix.perm.alloc(std::max<int64_t>(n, 1) * sizeof(uint32_t));
    int64_t nu = 0;
    if (n > 0) {
        k_flags<<<592, 256, 0, s>>>(key_hi, key_lo, leaf, n, flags.as<uint8_t>());
        BLSH_LAUNCH_CHECK();
        scan_exclusive_u8(flags.as<uint8_t>(), U.as<int64_t>(), n, scan, s);
        BLSH_CUDA(cudaMemcpyAsync(&nu, U.as<int64_t>() + n, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
        BLSH_CUDA(cudaStreamSynchronize(s));
    }
    ix.nu = nu;
    ix.ukey.alloc(std::max<int64_t>(nu, 1) * sizeof(Key128));
    ix.uleaf.alloc(std::max<int64_t>(nu, 1) * sizeof(int32_t));
    ix.uoff.alloc((std::max<int64_t>(nu, 1) + 1) * sizeof(uint32_t));
    BLSH_CUDA(cudaMemsetAsync(ix.uoff.p, 0, sizeof(uint32_t), s));
    if (n > 0) {
        k_unique<<<592, 256, 0, s>>>(key_hi, key_lo, leaf, id, flags.as<uint8_t>(), U.as<int64_t>(), n,
                                     ix.ukey.as<Key128>(), ix.uleaf.as<int32_t>(), ix.uoff.as<uint32_t>(),
                                     ix.perm.as<uint32_t>());
        BLSH_LAUNCH_CHECK();
    }
    ix.leaf_u.alloc((ix.G + 1) * sizeof(int64_t));
    k_leaf_u<<<(ix.G + 1 + 127) / 128, 128, 0, s>>>(ix.uleaf.as<int32_t>(), nu, ix.G, ix.leaf_u.as<int64_t>());
    BLSH_LAUNCH_CHECK();
    ix.leaf_u_h.assign(ix.G + 1, 0);
    BLSH_CUDA(cudaMemcpyAsync(ix.leaf_u_h.data(), ix.leaf_u.p, (ix.G + 1) * sizeof(int64_t), cudaMemcpyDeviceToHost, s));
    ix.Xp.alloc(std::max<int64_t>(n, 1) * ix.ds * sizeof(float));
    if (n > 0) {
        k_permute_rows<<<1184, 256, 0, s>>>(Xs, ix.ds, ix.perm.as<uint32_t>(), n, ix.Xp.as<float>());
        BLSH_LAUNCH_CHECK();
    }
    BLSH_CUDA(cudaStreamSynchronize(s));
}

}  // namespace blsh
