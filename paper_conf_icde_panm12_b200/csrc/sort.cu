// sort.cu -- b4: stable LSD radix sort of the bi-level code (leaf, Morton key)
// with the original id as payload ("linear array ... sorted to collect
// items with same LSH codes together").  8-bit digits, 18 digit positions
// (lo key 0-7, hi key 8-15, leaf 16-17); digits that are equal for every item
// are skipped after one OR/AND reduction pass.
#include "internal.cuh"

namespace blsh {

namespace {
constexpr int kSortThreads = 256;
constexpr int kSortWarps = kSortThreads / 32;
constexpr int kSortPer = 16;                       // items per thread
constexpr int kSortTile = kSortThreads * kSortPer;  // 4096 items per tile
constexpr int kWarpItems = 32 * kSortPer;           // 512 consecutive items per warp

__device__ __forceinline__ uint32_t digit_of(unsigned long long hi, unsigned long long lo,
                                             uint32_t leaf, int pass) {
    if (pass < 8) return (uint32_t)(lo >> (8 * pass)) & 255u;
    if (pass < 16) return (uint32_t)(hi >> (8 * (pass - 8))) & 255u;
    return (leaf >> (8 * (pass - 16))) & 255u;
}

__global__ void k_bits(const unsigned long long* __restrict__ hi, const unsigned long long* __restrict__ lo,
                       const uint32_t* __restrict__ leaf, int64_t n, unsigned long long* stats) {
    unsigned long long o_hi = 0, o_lo = 0, a_hi = ~0ull, a_lo = ~0ull;
    unsigned long long o_lf = 0, a_lf = ~0ull;
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n;
         i += (int64_t)gridDim.x * blockDim.x) {
        unsigned long long h = hi[i], l = lo[i], f = leaf[i];
        o_hi |= h; a_hi &= h; o_lo |= l; a_lo &= l; o_lf |= f; a_lf &= f;
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        o_hi |= __shfl_xor_sync(BLSH_FULL, o_hi, o);
        a_hi &= __shfl_xor_sync(BLSH_FULL, a_hi, o);
        o_lo |= __shfl_xor_sync(BLSH_FULL, o_lo, o);
        a_lo &= __shfl_xor_sync(BLSH_FULL, a_lo, o);
        o_lf |= __shfl_xor_sync(BLSH_FULL, o_lf, o);
        a_lf &= __shfl_xor_sync(BLSH_FULL, a_lf, o);
    }
    if ((threadIdx.x & 31) == 0) {
        atomicOr(&stats[0], o_hi); atomicAnd(&stats[1], a_hi);
        atomicOr(&stats[2], o_lo); atomicAnd(&stats[3], a_lo);
        atomicOr(&stats[4], o_lf); atomicAnd(&stats[5], a_lf);
    }
}

__global__ void __launch_bounds__(kSortThreads)
k_hist(const unsigned long long* __restrict__ hi, const unsigned long long* __restrict__ lo,
       const uint32_t* __restrict__ leaf, int64_t n, int pass, int64_t ntiles,
       int64_t* __restrict__ hist) {
    __shared__ uint32_t h[256];
    h[threadIdx.x] = 0;
    __syncthreads();
    const int64_t base = (int64_t)blockIdx.x * kSortTile;
    for (int i = threadIdx.x; i < kSortTile; i += kSortThreads) {
        const int64_t j = base + i;
        if (j < n) atomicAdd(&h[digit_of(hi[j], lo[j], leaf[j], pass)], 1u);
    }
    __syncthreads();
    hist[(int64_t)threadIdx.x * ntiles + blockIdx.x] = h[threadIdx.x];
}

__global__ void __launch_bounds__(kSortThreads)
k_scatter(const unsigned long long* __restrict__ hi, const unsigned long long* __restrict__ lo,
          const uint32_t* __restrict__ leaf, const uint32_t* __restrict__ id, int64_t n, int pass,
          int64_t ntiles, const int64_t* __restrict__ off, unsigned long long* __restrict__ hi_o,
          unsigned long long* __restrict__ lo_o, uint32_t* __restrict__ leaf_o,
          uint32_t* __restrict__ id_o) {
    __shared__ uint32_t cnt[kSortWarps][256];
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    for (int i = threadIdx.x; i < kSortWarps * 256; i += kSortThreads) (&cnt[0][0])[i] = 0;
    __syncthreads();
    const int64_t wbase = (int64_t)blockIdx.x * kSortTile + (int64_t)warp * kWarpItems;
    uint32_t packed[kSortPer];   // digit << 16 | rank within warp's digit run
#pragma unroll
    for (int r = 0; r < kSortPer; ++r) {
        const int64_t j = wbase + r * 32 + lane;
        const bool valid = j < n;
        const unsigned vm = __ballot_sync(BLSH_FULL, valid);
        uint32_t dg = valid ? digit_of(hi[j], lo[j], leaf[j], pass) : 256u + lane;
        const unsigned peers = __match_any_sync(BLSH_FULL, dg) & vm;
        uint32_t before = 0;
        if (valid) before = cnt[warp][dg];
        __syncwarp();
        if (valid && (peers & lanemask_lt()) == 0) cnt[warp][dg] = before + __popc(peers);
        __syncwarp();
        packed[r] = valid ? ((dg << 16) | (before + __popc(peers & lanemask_lt()))) : 0xFFFFFFFFu;
    }
    __syncthreads();
    {   // exclusive prefix over warps, per digit
        const int dgt = threadIdx.x;
        uint32_t run = 0;
#pragma unroll
        for (int w = 0; w < kSortWarps; ++w) {
            uint32_t c = cnt[w][dgt];
            cnt[w][dgt] = run;
            run += c;
        }
    }
    __syncthreads();
#pragma unroll
    for (int r = 0; r < kSortPer; ++r) {
        if (packed[r] == 0xFFFFFFFFu) continue;
        const int64_t j = wbase + r * 32 + lane;
        const uint32_t dg = packed[r] >> 16;
        const int64_t dst = off[(int64_t)dg * ntiles + blockIdx.x] + cnt[warp][dg] + (packed[r] & 0xFFFFu);
        hi_o[dst] = hi[j];
        lo_o[dst] = lo[j];
        leaf_o[dst] = leaf[j];
        id_o[dst] = id[j];
    }
}
}  // namespace

int radix_sort_entries(SortBufs& b, int64_t n, cudaStream_t s, int* passes_done) {
    *passes_done = 0;
    if (n <= 1) return 0;
    b.stats.ensure(8 * sizeof(unsigned long long));
    unsigned long long init[6] = {0ull, ~0ull, 0ull, ~0ull, 0ull, ~0ull};
    BLSH_CUDA(cudaMemcpyAsync(b.stats.p, init, sizeof(init), cudaMemcpyHostToDevice, s));
    k_bits<<<296, 256, 0, s>>>(b.hi[0].as<unsigned long long>(), b.lo[0].as<unsigned long long>(),
                               b.leaf[0].as<uint32_t>(), n, b.stats.as<unsigned long long>());
    BLSH_LAUNCH_CHECK();
    unsigned long long st[6];
    BLSH_CUDA(cudaMemcpyAsync(st, b.stats.p, sizeof(st), cudaMemcpyDeviceToHost, s));
    BLSH_CUDA(cudaStreamSynchronize(s));
    const int64_t ntiles = (n + kSortTile - 1) / kSortTile;
    b.hist.ensure((size_t)(256 * ntiles + 1) * sizeof(int64_t));
    int cur = 0;
    for (int pass = 0; pass < 18; ++pass) {
        unsigned long long o, a;
        int sh;
        if (pass < 8) { o = st[2]; a = st[3]; sh = 8 * pass; }
        else if (pass < 16) { o = st[0]; a = st[1]; sh = 8 * (pass - 8); }
        else { o = st[4]; a = st[5]; sh = 8 * (pass - 16); }
        if ((((o ^ a) >> sh) & 255ull) == 0) continue;   // digit constant over all items
        int64_t* hist = b.hist.as<int64_t>();
        k_hist<<<(unsigned)ntiles, kSortThreads, 0, s>>>(b.hi[cur].as<unsigned long long>(),
                                                         b.lo[cur].as<unsigned long long>(),
                                                         b.leaf[cur].as<uint32_t>(), n, pass, ntiles,
                                                         hist);
        BLSH_LAUNCH_CHECK();
        b.off.ensure((size_t)(256 * ntiles + 1) * sizeof(int64_t));
        scan_exclusive_i64(hist, b.off.as<int64_t>(), 256 * ntiles, b.scan, s);
        k_scatter<<<(unsigned)ntiles, kSortThreads, 0, s>>>(
            b.hi[cur].as<unsigned long long>(), b.lo[cur].as<unsigned long long>(),
            b.leaf[cur].as<uint32_t>(), b.id[cur].as<uint32_t>(), n, pass, ntiles,
            b.off.as<int64_t>(), b.hi[cur ^ 1].as<unsigned long long>(),
            b.lo[cur ^ 1].as<unsigned long long>(), b.leaf[cur ^ 1].as<uint32_t>(),
            b.id[cur ^ 1].as<uint32_t>());
        BLSH_LAUNCH_CHECK();
        cur ^= 1;
        ++*passes_done;
    }
    return cur;
}

}  // namespace blsh
