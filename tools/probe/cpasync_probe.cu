// Probe (experiment, not product): per-iteration cost of the screen producer's issue pattern on one SM:
// 128 threads x (8 x 16-byte cp.async [zero-fill or real] + cp.async.mbarrier.arrive.noinc), 384 iterations.
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdint>

__device__ __forceinline__ uint32_t su(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

__global__ void k(const char* src, int mode, int iters, long long* out) {
    extern __shared__ __align__(1024) unsigned char sm[];
    __shared__ __align__(8) uint64_t bar[8];
    const int t = threadIdx.x;
    if (t == 0) {
        for (int i = 0; i < 8; ++i) asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(su(&bar[i])), "r"(1 << 20));
        asm volatile("fence.mbarrier_init.release.cluster;");
    }
    __syncthreads();
    const long long t0 = clock64();
    for (int g = 0; g < iters; ++g) {
        const uint32_t dst = su(sm) + (uint32_t)((g & 7) * 16384) + t * 16;
        if (mode & 1) {
#pragma unroll
            for (int i = 0; i < 8; ++i) {
                const char* s = src + ((size_t)((g * 131 + i * 977 + t / 8 * 7919) % 100000)) * 768 + (t & 7) * 16;
                asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;" ::"r"(dst + 2048u * i), "l"(s), "r"((mode & 4) ? 16u : 0u) : "memory");
            }
        }
        if (mode & 2) asm volatile("cp.async.mbarrier.arrive.noinc.shared::cta.b64 [%0];" ::"r"(su(&bar[g & 7])) : "memory");
        else if (mode & 8) { asm volatile("cp.async.commit_group;"); asm volatile("cp.async.wait_group 6;"); }
    }
    asm volatile("cp.async.wait_all;" ::: "memory");
    __syncthreads();
    if (t == 0) out[blockIdx.x] = clock64() - t0;
}

int main() {
    char* src;
    cudaMalloc(&src, (size_t)100000 * 768);
    long long* out;
    cudaMalloc(&out, 148 * 8);
    cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, 8 * 16384);
    for (int mode : {0, 1, 2, 3, 5, 7, 9, 13}) {
        for (int blocks : {1, 148}) {
            k<<<blocks, 128, 8 * 16384>>>(src, mode, 384, out);
            cudaDeviceSynchronize();
            long long h[148];
            cudaMemcpy(h, out, blocks * 8, cudaMemcpyDeviceToHost);
            double m = 0;
            for (int i = 0; i < blocks; ++i) m += h[i];
            printf("mode %2d (%s%s%s%s) blocks %3d: %.0f cycles per iteration\n", mode, (mode & 1) ? "copies " : "",
                   (mode & 4) ? "real " : ((mode & 1) ? "zero-fill " : ""), (mode & 2) ? "arrive.noinc " : "",
                   (mode & 8) ? "wait_group " : "", blocks, m / blocks / 384);
        }
    }
    printf("%s\n", cudaGetErrorString(cudaGetLastError()));
    return 0;
}
