// hashcore.cuh -- device pieces of the hash that data (b3) and queries (a2) share:
// the E8 decoder of Eq. 6 with the tie-breaks of R14, and code -> key.
#pragma once

#include "common.cuh"

namespace blsh {

// Nearest point of D8 (integer vectors with even coordinate sum) to w (R14).
__device__ __forceinline__ void d8_nearest(const float* w, int32_t* z) {
    int32_t sum = 0;
#pragma unroll
    for (int j = 0; j < 8; ++j) {
        z[j] = (int32_t)rintf(w[j]);   // round half to even
        sum += z[j];
    }
    if (sum & 1) {
        int jb = 0;
        float best = -1.0f;
#pragma unroll
        for (int j = 0; j < 8; ++j) {
            const float dev = fabsf(__fsub_rn(w[j], (float)z[j]));
            if (dev > best) { best = dev; jb = j; }
        }
        float r = 0.0f;
#pragma unroll
        for (int j = 0; j < 8; ++j)
            if (j == jb) r = __fsub_rn(w[j], (float)z[j]);
#pragma unroll
        for (int j = 0; j < 8; ++j)
            if (j == jb) z[j] += (r >= 0.0f) ? 1 : -1;
    }
}

// fp64 squared distance from y to the doubled E8 point c2/2 (fma-accumulated, ascending j).
__device__ __forceinline__ double e8_dist2(const float* y, const int32_t* c2) {
    double s = 0.0;
#pragma unroll
    for (int j = 0; j < 8; ++j) {
        const double e = __dsub_rn((double)y[j], __dmul_rn(0.5, (double)c2[j]));
        s = __fma_rn(e, e, s);
    }
    return s;
}

// E8 DECODE (Eq. 6): nearest E8 point in doubled coordinates.
__device__ __forceinline__ void e8_decode(const float* y, int32_t* c2) {
    int32_t z0[8], z1[8], a[8], b[8];
    float w[8];
    d8_nearest(y, z0);
#pragma unroll
    for (int j = 0; j < 8; ++j) w[j] = __fsub_rn(y[j], 0.5f);
    d8_nearest(w, z1);
#pragma unroll
    for (int j = 0; j < 8; ++j) {
        a[j] = 2 * z0[j];
        b[j] = 2 * z1[j] + 1;
    }
    const double d0 = e8_dist2(y, a), d1 = e8_dist2(y, b);
    const bool pick_b = d1 < d0;   // ties -> integer coset
#pragma unroll
    for (int j = 0; j < 8; ++j) c2[j] = pick_b ? b[j] : a[j];
}

// Quantise the projections t[M] (Z^M floor or E8) into a code inside the
// Morton range; returns false when the code leaves the range (R9, R14).
// On false, `code` holds the clamped floor (Z^M) or zeros (E8).
__device__ __forceinline__ bool quantise(const float* t, int M, int B, int quantizer, int32_t* code) {
    bool ok = true;
    if (quantizer == 0) {
        const float lo = -(float)(1 << (B - 1)), hi = (float)((1 << (B - 1)) - 1);
        for (int i = 0; i < M; ++i) {
            const float f = floorf(t[i]);
            const float c = f < lo ? lo : (f > hi ? hi : f);
            if (c != f) ok = false;
            code[i] = (int32_t)c;
        }
    } else if (M != 8 && M != 16) {
        ok = false;
    } else {   // E8 (Eq. 6); M = 16: two E8 blocks decoded independently (R28)
        for (int i = 0; i < M; ++i)
            if (!(fabsf(t[i]) < 16000.0f)) ok = false;
        if (ok) {
            for (int blk = 0; blk < M / 8; ++blk) e8_decode(t + 8 * blk, code + 8 * blk);
            const int32_t lo = -(1 << (B - 1)), hi = (1 << (B - 1)) - 1;
            for (int i = 0; i < M; ++i)
                if (code[i] < lo || code[i] > hi) ok = false;
        }
        if (!ok)
            for (int i = 0; i < M; ++i) code[i] = 0;
    }
    return ok;
}

// A warp's [32 rows x 32 columns] chunks of fp32 rows (row pitch ds floats, ds % 4 == 0),
// staged through registers into shared memory tile[r * kRowPitch + c]: coalesced 16-byte
// loads (8 lanes per row's 128-byte chunk, 4 rows per instruction), rows qid(0..nrow-1),
// zeros beyond.  load(j0) issues the 8 loads of chunk j0 into registers (the next chunk's
// loads are in flight while the current one is consumed), store() writes them to the tile.
// Read back by lane = row, the 16-byte reads of 8 lanes fall in distinct bank groups (pitch 36).
constexpr int kRowPitch = 36;
struct ChunkStager {
    float4 v[8];
    template <class QID>
    __device__ __forceinline__ void load(const float* __restrict__ Q, int ds, QID qid, int nrow, int j0, int lane) {
        const int c4 = lane & 7, rr = lane >> 3;
        const int col = j0 + 4 * c4;
#pragma unroll
        for (int r4 = 0; r4 < 8; ++r4) {
            const int r = 4 * r4 + rr;
            // streaming loads (evict-first): a row chunk is read once per pass, L1 keeps the
            // parameters (tree nodes, A_g) the chains read again and again
            v[r4] = (r < nrow && col < ds) ? __ldcs(reinterpret_cast<const float4*>(Q + (size_t)qid(r) * ds + col))
                                           : make_float4(0.f, 0.f, 0.f, 0.f);
        }
    }
    __device__ __forceinline__ void store(float* tile, int lane) const {
        const int c4 = lane & 7, rr = lane >> 3;
#pragma unroll
        for (int r4 = 0; r4 < 8; ++r4) *reinterpret_cast<float4*>(tile + (4 * r4 + rr) * kRowPitch + 4 * c4) = v[r4];
    }
};

}  // namespace blsh
