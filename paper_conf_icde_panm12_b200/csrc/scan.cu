// scan.cu -- device exclusive prefix sums (three-phase: reduce, scan partials, scan+add).
#include "internal.cuh"

namespace blsh {

namespace {
constexpr int kScanThreads = 1024;
constexpr int kScanPer = 4;
constexpr int kScanTile = kScanThreads * kScanPer;

__device__ __forceinline__ int64_t block_exclusive(int64_t v, int64_t* smem_warp, int64_t& total) {
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    int64_t x = v;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        int64_t y = __shfl_up_sync(BLSH_FULL, x, o);
        if (lane >= o) x += y;
    }
    if (lane == 31) smem_warp[warp] = x;
    __syncthreads();
    if (warp == 0) {
        int64_t w = lane < (int)(blockDim.x >> 5) ? smem_warp[lane] : 0;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            int64_t y = __shfl_up_sync(BLSH_FULL, w, o);
            if (lane >= o) w += y;
        }
        smem_warp[lane] = w;   // inclusive per warp
    }
    __syncthreads();
    const int64_t warp_off = warp ? smem_warp[warp - 1] : 0;
    total = smem_warp[(blockDim.x >> 5) - 1];
    return warp_off + x - v;
}

template <typename T>
__global__ void __launch_bounds__(kScanThreads) k_scan_reduce(const T* __restrict__ in, int64_t n,
                                                              int64_t* __restrict__ bsum) {
    __shared__ int64_t sw[32];
    const int64_t base = (int64_t)blockIdx.x * kScanTile + (int64_t)threadIdx.x * kScanPer;
    int64_t s = 0;
#pragma unroll
    for (int i = 0; i < kScanPer; ++i)
        if (base + i < n) s += (int64_t)in[base + i];
    int64_t tot;
    block_exclusive(s, sw, tot);
    if (threadIdx.x == 0) bsum[blockIdx.x] = tot;
}

__global__ void __launch_bounds__(kScanThreads) k_scan_partials(int64_t* bsum, int64_t nb) {
    __shared__ int64_t sw[32];
    const int64_t per = (nb + kScanThreads - 1) / kScanThreads;
    const int64_t lo = (int64_t)threadIdx.x * per;
    int64_t s = 0;
    for (int64_t i = lo; i < lo + per && i < nb; ++i) s += bsum[i];
    int64_t tot;
    int64_t ex = block_exclusive(s, sw, tot);
    for (int64_t i = lo; i < lo + per && i < nb; ++i) {
        int64_t v = bsum[i];
        bsum[i] = ex;
        ex += v;
    }
    if (threadIdx.x == 0) bsum[nb] = tot;
}

template <typename T>
__global__ void __launch_bounds__(kScanThreads) k_scan_final(const T* __restrict__ in, int64_t n,
                                                             const int64_t* __restrict__ bsum,
                                                             int64_t nb, int64_t* __restrict__ out) {
    __shared__ int64_t sw[32];
    const int64_t base = (int64_t)blockIdx.x * kScanTile + (int64_t)threadIdx.x * kScanPer;
    int64_t v[kScanPer];
    int64_t s = 0;
#pragma unroll
    for (int i = 0; i < kScanPer; ++i) {
        v[i] = base + i < n ? (int64_t)in[base + i] : 0;
        s += v[i];
    }
    int64_t tot;
    int64_t ex = block_exclusive(s, sw, tot) + bsum[blockIdx.x];
#pragma unroll
    for (int i = 0; i < kScanPer; ++i) {
        if (base + i < n) out[base + i] = ex;
        ex += v[i];
    }
    if (blockIdx.x == 0 && threadIdx.x == 0) out[n] = bsum[nb];
}

template <typename T>
void scan_impl(const T* in, int64_t* out, int64_t n, ScanTemp& t, cudaStream_t s) {
    const int64_t nb = (n + kScanTile - 1) / kScanTile;
    const int64_t nbb = nb > 0 ? nb : 1;
    t.blocks.ensure((size_t)(nbb + 1) * sizeof(int64_t));
    int64_t* bs = t.blocks.as<int64_t>();
    if (n == 0) {
        BLSH_CUDA(cudaMemsetAsync(out, 0, sizeof(int64_t), s));
        return;
    }
    k_scan_reduce<T><<<(unsigned)nb, kScanThreads, 0, s>>>(in, n, bs);
    BLSH_LAUNCH_CHECK();
    k_scan_partials<<<1, kScanThreads, 0, s>>>(bs, nb);
    BLSH_LAUNCH_CHECK();
    k_scan_final<T><<<(unsigned)nb, kScanThreads, 0, s>>>(in, n, bs, nb, out);
    BLSH_LAUNCH_CHECK();
}
}  // namespace

void scan_exclusive_i64(const int64_t* in, int64_t* out, int64_t n, ScanTemp& t, cudaStream_t s) {
    scan_impl<int64_t>(in, out, n, t, s);
}
void scan_exclusive_u8(const uint8_t* in, int64_t* out, int64_t n, ScanTemp& t, cudaStream_t s) {
    scan_impl<uint8_t>(in, out, n, t, s);
}

}  // namespace blsh
