// resid.cu -- the short-list screen's compact copy of the table (a5, DESIGN.md §7
// "The short-list (a5) on B200").
//
// The table rows Xp (fp32, table order) are cut into anchor blocks of 2^kAnchorShift
// consecutive rows.  Per block b: the anchor a_b (fp32 mean of its rows, fp64 sums),
// a power-of-two scale s_b with max |x - a_b| / s_b in [2^14, 2^15), and per row the
// fp16 residual r = fp16_rn((x - a_b) / s_b), padded with zeros to dr (a multiple of
// 64) columns.  x~ = a_b + s_b r is the screen's stand-in for x; per row the library
// keeps, from fp64 sums,
//   nu  = |s_b r|^2,  rho = a_b . (s_b r) (diagnostic),  n = |s_b r| (rounded up),
//   G   = the row's share of the screen's error bound (rounding of nu, the
//         distance between x and x~: 4097 |x - x~|^2 for the 2^-12 AM-GM split, and
//         2^-13 n^2 for the K table's relative error),
// so the screen never needs the fp32 row: it reads 2 bytes per coordinate, and the
// exact fp32 rows are only read by the rescoring of its survivors.  The anchors do
// not have to be good for correctness (every bound carries |s_b r| and |x - x~|);
// Morton-consecutive rows of one leaf are close, so |s_b r| is about a cluster radius.
#include <algorithm>

#include <cuda_fp16.h>

#include "internal.cuh"

namespace blsh {

namespace {

constexpr int kAT = 256;

__device__ __forceinline__ double warp_sum_d(double v) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(BLSH_FULL, v, o);
    return v;
}

__global__ void __launch_bounds__(kAT) k_anchor_rows(const float* __restrict__ Xp, int64_t n, int ds, int dr,
                                                     float* __restrict__ anc, float* __restrict__ bscale,
                                                     __half* __restrict__ Rh, float4* __restrict__ rconst) {
    extern __shared__ float a32[];          // [dr] the block's anchor
    __shared__ double red[kAT / 32];
    __shared__ float s_scale;
    __shared__ double s_anorm;
    const int64_t b = blockIdx.x;
    const int64_t r0 = b << kAnchorShift;
    const int nr = (int)min((int64_t)1 << kAnchorShift, n - r0);
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    // anchor: fp64 column sums over the block's rows in row order
    for (int c = threadIdx.x; c < dr; c += kAT) {
        double s = 0.0;
        if (c < ds)
            for (int r = 0; r < nr; ++r) s += (double)Xp[(size_t)(r0 + r) * ds + c];
        const float a = c < ds ? (float)(s / (double)nr) : 0.0f;
        a32[c] = a;
        anc[(size_t)b * dr + c] = a;
    }
    __syncthreads();
    // block scale: largest |x - a| over the block
    double mx = 0.0, an = 0.0;
    for (int c = threadIdx.x; c < ds; c += kAT) {
        const double a = (double)a32[c];
        an += a * a;
        for (int r = 0; r < nr; ++r) mx = fmax(mx, fabs((double)Xp[(size_t)(r0 + r) * ds + c] - a));
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) mx = fmax(mx, __shfl_xor_sync(BLSH_FULL, mx, o));
    an = warp_sum_d(an);
    if (lane == 0) red[warp] = mx;
    __syncthreads();
    if (threadIdx.x == 0) {
        double m = 0.0;
        for (int w = 0; w < kAT / 32; ++w) m = fmax(m, red[w]);
        int e = 0;
        if (m > 0.0) { frexp(m, &e); e -= 15; }   // m / 2^e in [2^14, 2^15)
        e = max(-120, min(120, e));
        s_scale = ldexpf(1.0f, e);
        bscale[b] = s_scale;
    }
    __syncthreads();
    if (lane == 0) red[warp] = an;
    __syncthreads();
    if (threadIdx.x == 0) {
        double t = 0.0;
        for (int w = 0; w < kAT / 32; ++w) t += red[w];
        s_anorm = sqrt(t);
    }
    __syncthreads();
    const double sc = (double)s_scale;
    const double anorm = s_anorm;
    // residual rows: one warp per row
    for (int r = warp; r < nr; r += kAT / 32) {
        const int64_t row = r0 + r;
        const float* x = Xp + (size_t)row * ds;
        __half* out = Rh + (size_t)row * dr;
        double nu = 0.0, rho = 0.0, e2 = 0.0;
        for (int c = lane; c < dr; c += 32) {
            __half h = __float2half_rn(0.0f);
            if (c < ds) {
                const double a = (double)a32[c];
                const double diff = (double)x[c] - a;          // exact (two fp32 values)
                h = __double2half(diff / sc);                   // round to nearest (power-of-two scale)
                const double rr = (double)__half2float(h) * sc;
                nu += rr * rr;
                rho += a * rr;
                const double ex = diff - rr;
                e2 += ex * ex;
            }
            out[c] = h;
        }
        nu = warp_sum_d(nu);
        rho = warp_sum_d(rho);
        e2 = warp_sum_d(e2);
        if (lane == 0) {
            const double nrm = sqrt(nu) * (1.0 + 0x1p-40);
            const double G = 0x1p-23 * nu + 4097.0 * e2 * (1.0 + 0x1p-20) + 0x1p-13 * nu;
            float4 v;
            v.x = (float)nu;
            v.y = (float)rho;
            v.z = __double2float_ru(nrm);
            v.w = __double2float_ru(G * (1.0 + 0x1p-20));
            rconst[row] = v;
        }
    }
}

}  // namespace

int screen_cols(int ds) { return (ds + 63) & ~63; }

void build_screen_rows(blsh_index& ix, cudaStream_t s) {
    const int64_t n = ix.n_owned;
    const int dr = screen_cols(ix.ds);
    ix.dr = dr;
    const int64_t nblk = (n + (1 << kAnchorShift) - 1) >> kAnchorShift;
    ix.nanchor = nblk;
    ix.anc.alloc((size_t)std::max<int64_t>(nblk, 1) * dr * sizeof(float));
    ix.bscale.alloc((size_t)std::max<int64_t>(nblk, 1) * sizeof(float));
    ix.Rh.alloc((size_t)std::max<int64_t>(n, 1) * dr * sizeof(__half));
    ix.rconst.alloc((size_t)std::max<int64_t>(n, 1) * sizeof(float4));
    if (n == 0) return;
    const size_t smem = (size_t)dr * sizeof(float);
    BLSH_CUDA(cudaFuncSetAttribute(k_anchor_rows, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    k_anchor_rows<<<(unsigned)nblk, kAT, smem, s>>>(ix.Xp.as<float>(), n, ix.ds, dr, ix.anc.as<float>(),
                                                    ix.bscale.as<float>(), ix.Rh.as<__half>(), ix.rconst.as<float4>());
    BLSH_LAUNCH_CHECK();
}

}  // namespace blsh
