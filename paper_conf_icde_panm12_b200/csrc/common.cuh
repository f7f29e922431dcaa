// common.cuh -- device helpers shared by the library's kernels (not by the oracle).
//
// Canonical arithmetic (R1): every floating-point operation that
// decides an integer (hash code, tree side, median, probe order) is written
// with an explicit round-to-nearest intrinsic so that nvcc can never contract
// or reorder it.
#pragma once

#include <cstdint>
#include <cstring>
#include <cuda_runtime.h>

#define BLSH_WARP 32
#define BLSH_FULL 0xffffffffu

namespace blsh {

struct Key128 {
    unsigned long long hi, lo;
};

__host__ __device__ __forceinline__ bool key_lt(const Key128& a, const Key128& b) {
    return a.hi < b.hi || (a.hi == b.hi && a.lo < b.lo);
}
__host__ __device__ __forceinline__ bool key_le(const Key128& a, const Key128& b) {
    return a.hi < b.hi || (a.hi == b.hi && a.lo <= b.lo);
}
__host__ __device__ __forceinline__ bool key_eq(const Key128& a, const Key128& b) {
    return a.hi == b.hi && a.lo == b.lo;
}

// Bits per coordinate of the Morton key (R9).
__host__ __device__ __forceinline__ int bits_per_coord(int M) {
    int B = 128 / M;
    return B > 24 ? 24 : B;
}

// Morton interleave (R9): bit p of u_i = code_i + 2^(B-1) goes to key
// bit p*M + (M-1-i).  Caller guarantees the code is inside the range.
// Bits 0..7 of b to bit 0 of bytes 0..7 (multiply-replicate, mask bit j of
// byte j, carry it to bit 7 with +0x7F, which never carries across bytes).
__device__ __forceinline__ unsigned long long spread8(uint32_t b) {
    const unsigned long long r = ((unsigned long long)(b & 0xFFu) * 0x0101010101010101ull) & 0x8040201008040201ull;
    return ((r + 0x7F7F7F7F7F7F7F7Full) & 0x8080808080808080ull) >> 7;
}

__device__ __forceinline__ Key128 morton_key(const int32_t* code, int M, int B) {
    unsigned long long hi = 0ull, lo = 0ull;
    const int off = 1 << (B - 1);
    if (M == 8 && B == 16) {   // bit p of u_i -> key byte p, bit 7-i: the same interleave, 2 spreads per coordinate
#pragma unroll
        for (int i = 0; i < 8; ++i) {
            const uint32_t u = (uint32_t)(code[i] + off);
            lo |= spread8(u) << (7 - i);
            hi |= spread8(u >> 8) << (7 - i);
        }
        return Key128{hi, lo};
    }
    for (int i = 0; i < M; ++i) {
        uint32_t u = (uint32_t)(code[i] + off);
        const int base = M - 1 - i;
        for (int p = 0; p < B; ++p) {
            unsigned long long bit = (u >> p) & 1u;
            int pos = p * M + base;
            if (pos < 64) lo |= bit << pos;
            else hi |= bit << (pos - 64);
        }
    }
    return Key128{hi, lo};
}

// Total order of fp32 values as u32 (R5).
__host__ __device__ __forceinline__ uint32_t fkey(float f) {
#ifdef __CUDA_ARCH__
    uint32_t u = __float_as_uint(f);
#else
    uint32_t u;
    memcpy(&u, &f, 4);
#endif
    return (u & 0x80000000u) ? ~u : (u | 0x80000000u);
}
__device__ __forceinline__ float fkey_inv(uint32_t k) {
    uint32_t u = (k & 0x80000000u) ? (k & 0x7FFFFFFFu) : ~k;
    return __uint_as_float(u);
}

// Packed short-list entry: (fp32 bits of d^2) << 32 | id32.  For d^2 >= 0 the
// integer order is the (d^2, id) order.  EMPTY sorts after every real entry.
constexpr unsigned long long kEmpty = 0xFFFFFFFFFFFFFFFFull;
constexpr unsigned long long kPadPacked = 0x7F800000FFFFFFFFull;

__device__ __forceinline__ unsigned long long pack_entry(float d2, uint32_t id) {
    return ((unsigned long long)__float_as_uint(d2) << 32) | id;
}

__device__ __forceinline__ unsigned lanemask_lt() {
    unsigned m;
    asm("mov.u32 %0, %%lanemask_lt;" : "=r"(m));
    return m;
}

template <typename T>
__device__ __forceinline__ T ldg(const T* p) { return __ldg(p); }

}  // namespace blsh
