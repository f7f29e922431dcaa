// resid.cu -- the short-list screen's compact copy of the table (a5, DESIGN.md §7
// "The short-list (a5) on B200").
//
// The table rows Xp (fp32, table order) are cut into anchor GROUPS: maximal runs of
// consecutive buckets of one leaf whose consecutive bucket means lie within tau of each
// other (tau = 4 x the median RMS radius of the buckets with >= 2 rows), so a group is a
// run of neighbouring cells of one cluster (a fixed number of Morton-consecutive rows is
// not: the Z-curve interleaves the cells of different clusters).  Per group g: the anchor
// a_g (fp32 mean of its rows, fp64 sums), a power-of-two scale s_g with
// max |x - a_g| / s_g in [2^14, 2^15), and per row the fp16 residual
// r = fp16_rn((x - a_g) / s_g), padded with zeros to dr (a multiple of 64) columns.
// Layout of the fp16 rows ("atoms"): table rows 8a..8a+7 form atom a; panel-major: for every
// 64-column panel p the atoms are consecutive KBs (panel p, atom a at (p * atoms + a) KB), an
// atom's 8 x 128 bytes with 16-byte chunk ch of row r stored at chunk ch ^ r -- the
// 128-byte-swizzled K-major layout the tensor core reads from shared memory.  A run of
// consecutive table rows (a bucket) is then one contiguous bulk copy per panel, with no
// per-16-byte copies and no swizzling on the device.
// x~ = a_g + s_g r is the screen's stand-in for x; per row the library keeps, from fp64
// sums,
//   nu = |s_g r|^2,  s_g,  n = |s_g r| (rounded up),
//   G  = the row's share of the screen's error bound (rounding of nu, the distance between
//        x and x~: 4097 |x - x~|^2 for the 2^-12 AM-GM split, and 2^-13 n^2 for the K
//        table's relative error),
// so the screen never needs the fp32 row: it reads 2 bytes per coordinate, and the exact
// fp32 rows are only read by the rescoring of its survivors.  The grouping only affects
// how tight the screen's bound is (every bound carries |s_g r| and |x - x~|), never a result.
#include <algorithm>
#include <vector>

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

// One warp per bucket: fp32 mean (fp64 sums) and mean squared distance to it.
__global__ void __launch_bounds__(256) k_bucket_stats(const float* __restrict__ Xp, int ds,
                                                      const uint32_t* __restrict__ uoff, int64_t nu,
                                                      float* __restrict__ bmean, float* __restrict__ br2) {
    const int lane = threadIdx.x & 31;
    const int64_t u = blockIdx.x * (int64_t)8 + (threadIdx.x >> 5);
    if (u >= nu) return;
    const int64_t r0 = uoff[u], r1 = uoff[u + 1];
    const double inv = 1.0 / (double)(r1 - r0);
    double m2 = 0.0;
    for (int c0 = 0; c0 < ds; c0 += 32) {
        const int c = c0 + lane;
        double s = 0.0;
        if (c < ds)
            for (int64_t r = r0; r < r1; ++r) s += (double)Xp[(size_t)r * ds + c];
        const float m = (float)(s * inv);
        if (c < ds) {
            bmean[(size_t)u * ds + c] = m;
            for (int64_t r = r0; r < r1; ++r) {
                const double e = (double)Xp[(size_t)r * ds + c] - (double)m;
                m2 += e * e;
            }
        }
    }
    m2 = warp_sum_d(m2);
    if (lane == 0) br2[u] = (float)(m2 * inv);
}

// Group starts: the first bucket of every leaf, and every bucket whose mean is more than
// tau from the previous bucket's.  One warp per bucket.
__global__ void __launch_bounds__(256) k_group_flags(const float* __restrict__ bmean, int ds,
                                                     const int32_t* __restrict__ uleaf, int64_t nu, float tau2,
                                                     uint8_t* __restrict__ flag) {
    const int lane = threadIdx.x & 31;
    const int64_t u = blockIdx.x * (int64_t)8 + (threadIdx.x >> 5);
    if (u >= nu) return;
    if (u == 0 || uleaf[u] != uleaf[u - 1]) {
        if (lane == 0) flag[u] = 1;
        return;
    }
    float s = 0.f;
    for (int c = lane; c < ds; c += 32) {
        const float e = bmean[(size_t)u * ds + c] - bmean[(size_t)(u - 1) * ds + c];
        s = fmaf(e, e, s);
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(BLSH_FULL, s, o);
    if (lane == 0) flag[u] = s > tau2 ? 1 : 0;
}

// Group of every table row and the first row of every group.
__global__ void k_group_rows(const uint8_t* __restrict__ flag, const int64_t* __restrict__ gex,
                             const uint32_t* __restrict__ uoff, int64_t nu, uint32_t* __restrict__ rgrp,
                             int64_t* __restrict__ gstart) {
    const int64_t u = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (u >= nu) return;
    const int64_t g = gex[u] + flag[u] - 1;
    if (flag[u]) gstart[g] = uoff[u];
    if (u == nu - 1) gstart[g + 1] = uoff[nu];
    for (uint32_t r = uoff[u]; r < uoff[u + 1]; ++r) rgrp[r] = (uint32_t)g;
}

// One CTA per group: anchor, scale, fp16 residual rows, per-row bound constants.
__global__ void __launch_bounds__(kAT) k_anchor_rows(const float* __restrict__ Xp, const int64_t* __restrict__ gstart,
                                                     int ds, int dr, int64_t natom, float* __restrict__ anc,
                                                     __half* __restrict__ Rh, float4* __restrict__ rconst) {
    extern __shared__ float a32[];          // [dr] the group's anchor
    __shared__ double red[kAT / 32];
    __shared__ float s_scale;
    const int64_t g = blockIdx.x;
    const int64_t r0 = gstart[g];
    const int64_t nr = gstart[g + 1] - r0;
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    // anchor: fp64 column sums over the group's rows in row order
    for (int c = threadIdx.x; c < dr; c += kAT) {
        double s = 0.0;
        if (c < ds)
            for (int64_t r = 0; r < nr; ++r) s += (double)Xp[(size_t)(r0 + r) * ds + c];
        const float a = c < ds ? (float)(s / (double)nr) : 0.0f;
        a32[c] = a;
        anc[(size_t)g * dr + c] = a;
    }
    __syncthreads();
    // scale: largest |x - a| over the group
    double mx = 0.0;
    for (int c = threadIdx.x; c < ds; c += kAT) {
        const double a = (double)a32[c];
        for (int64_t r = 0; r < nr; ++r) mx = fmax(mx, fabs((double)Xp[(size_t)(r0 + r) * ds + c] - a));
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) mx = fmax(mx, __shfl_xor_sync(BLSH_FULL, mx, o));
    if (lane == 0) red[warp] = mx;
    __syncthreads();
    if (threadIdx.x == 0) {
        double m = 0.0;
        for (int w = 0; w < kAT / 32; ++w) m = fmax(m, red[w]);
        int e = 0;
        if (m > 0.0) { frexp(m, &e); e -= 15; }   // m / 2^e in [2^14, 2^15)
        e = max(-120, min(120, e));
        s_scale = ldexpf(1.0f, e);
    }
    __syncthreads();
    const double sc = (double)s_scale;
    // residual rows: one warp per row
    for (int64_t r = warp; r < nr; r += kAT / 32) {
        const int64_t row = r0 + r;
        const float* x = Xp + (size_t)row * ds;
        // panel c >> 6, atom (row >> 3), row (row & 7), chunk ((c >> 3) & 7) ^ (row & 7), element c & 7
        __half* out = Rh + (size_t)(row >> 3) * 512 + (row & 7) * 64;
        const int sw = (int)(row & 7);
        double nu = 0.0, e2 = 0.0;
        for (int c = lane; c < dr; c += 32) {
            __half h = __float2half_rn(0.0f);
            if (c < ds) {
                const double a = (double)a32[c];
                const double diff = (double)x[c] - a;          // exact (two fp32 values)
                h = __double2half(diff / sc);                   // round to nearest (power-of-two scale)
                const double rr = (double)__half2float(h) * sc;
                nu += rr * rr;
                const double ex = diff - rr;
                e2 += ex * ex;
            }
            out[(size_t)(c >> 6) * natom * 512 + ((((c >> 3) & 7) ^ sw) << 3) + (c & 7)] = h;
        }
        nu = warp_sum_d(nu);
        e2 = warp_sum_d(e2);
        if (lane == 0) {
            const double nrm = sqrt(nu) * (1.0 + 0x1p-40);
            const double G = 0x1p-23 * nu + 4097.0 * e2 * (1.0 + 0x1p-20) + 0x1p-13 * nu;
            float4 v;
            v.x = (float)nu;
            v.y = s_scale;
            v.z = __double2float_ru(nrm);
            v.w = __double2float_ru(G * (1.0 + 0x1p-20));
            rconst[row] = v;
        }
    }
}

}  // namespace

int screen_cols(int ds) { return (ds + 63) & ~63; }

void build_screen_rows(blsh_index& ix, cudaStream_t s) {
    const int64_t n = ix.n_owned, nu = ix.nu;
    const int ds = ix.ds, dr = screen_cols(ds);
    ix.dr = dr;
    const int64_t natom = (n + 7) / 8;   // rows padded to whole atoms (zero rows)
    ix.Rh.alloc((size_t)std::max<int64_t>(natom, 1) * 8 * dr * sizeof(__half));
    BLSH_CUDA(cudaMemsetAsync(ix.Rh.p, 0, (size_t)std::max<int64_t>(natom, 1) * 8 * dr * sizeof(__half), s));
    ix.rconst.alloc((size_t)std::max<int64_t>(natom, 1) * 8 * sizeof(float4));
    BLSH_CUDA(cudaMemsetAsync(ix.rconst.p, 0, (size_t)std::max<int64_t>(natom, 1) * 8 * sizeof(float4), s));
    ix.rgrp.alloc((size_t)std::max<int64_t>(n, 1) * sizeof(uint32_t));
    if (n == 0 || nu == 0) {
        ix.nanchor = 0;
        ix.anc.alloc(dr * sizeof(float));
        ix.gstart.alloc(2 * sizeof(int64_t));
        BLSH_CUDA(cudaMemsetAsync(ix.gstart.p, 0, 2 * sizeof(int64_t), s));
        return;
    }
    // bucket means and radii
    DevBuf bmean, br2, flag, gex;
    bmean.alloc((size_t)nu * ds * sizeof(float));
    br2.alloc((size_t)nu * sizeof(float));
    const unsigned gw = (unsigned)((nu + 7) / 8);
    k_bucket_stats<<<gw, 256, 0, s>>>(ix.Xp.as<float>(), ds, ix.uoff.as<uint32_t>(), nu, bmean.as<float>(),
                                      br2.as<float>());
    BLSH_LAUNCH_CHECK();
    // tau = 4 x the median RMS radius of the buckets with >= 2 rows (0 if there are none)
    std::vector<float> r2(nu);
    std::vector<uint32_t> uo(nu + 1);
    BLSH_CUDA(cudaMemcpyAsync(r2.data(), br2.p, nu * sizeof(float), cudaMemcpyDeviceToHost, s));
    BLSH_CUDA(cudaMemcpyAsync(uo.data(), ix.uoff.p, (nu + 1) * sizeof(uint32_t), cudaMemcpyDeviceToHost, s));
    BLSH_CUDA(cudaStreamSynchronize(s));
    std::vector<float> multi;
    multi.reserve(nu);
    for (int64_t u = 0; u < nu; ++u)
        if (uo[u + 1] - uo[u] >= 2) multi.push_back(r2[u]);
    float med = 0.f;
    if (!multi.empty()) {
        std::nth_element(multi.begin(), multi.begin() + (multi.size() - 1) / 2, multi.end());
        med = multi[(multi.size() - 1) / 2];
    }
    const float tau2 = 16.0f * med;
    ix.anchor_tau2 = tau2;
    flag.alloc((size_t)nu);
    gex.alloc((size_t)(nu + 1) * sizeof(int64_t));
    k_group_flags<<<gw, 256, 0, s>>>(bmean.as<float>(), ds, ix.uleaf.as<int32_t>(), nu, tau2, flag.as<uint8_t>());
    BLSH_LAUNCH_CHECK();
    ScanTemp st;
    scan_exclusive_u8(flag.as<uint8_t>(), gex.as<int64_t>(), nu, st, s);
    int64_t ng = 0;
    BLSH_CUDA(cudaMemcpyAsync(&ng, gex.as<int64_t>() + nu, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
    BLSH_CUDA(cudaStreamSynchronize(s));
    ix.nanchor = ng;
    ix.gstart.alloc((size_t)(ng + 1) * sizeof(int64_t));
    k_group_rows<<<(unsigned)((nu + 255) / 256), 256, 0, s>>>(flag.as<uint8_t>(), gex.as<int64_t>(),
                                                              ix.uoff.as<uint32_t>(), nu, ix.rgrp.as<uint32_t>(),
                                                              ix.gstart.as<int64_t>());
    BLSH_LAUNCH_CHECK();
    ix.anc.alloc((size_t)ng * dr * sizeof(float));
    const size_t smem = (size_t)dr * sizeof(float);
    BLSH_CUDA(cudaFuncSetAttribute(k_anchor_rows, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    k_anchor_rows<<<(unsigned)ng, kAT, smem, s>>>(ix.Xp.as<float>(), ix.gstart.as<int64_t>(), ds, dr, natom,
                                                   ix.anc.as<float>(), ix.Rh.as<__half>(), ix.rconst.as<float4>());
    BLSH_LAUNCH_CHECK();
    BLSH_CUDA(cudaStreamSynchronize(s));
}

}  // namespace blsh
