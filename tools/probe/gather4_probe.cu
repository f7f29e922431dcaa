// Probe (experiment, not product): does cp.async.bulk.tensor ... tile::gather4 load 4 arbitrary rows of a
// 2-D fp16 tensor into 128-byte-swizzled shared memory, and which box height does the tensor map need?
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -o /tmp/g4 tools/probe/gather4_probe.cu -lcuda
#include <cuda.h>
#include <cuda_fp16.h>
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdint>
#include <vector>

__global__ void k(const __grid_constant__ CUtensorMap tm, int r0, int r1, int r2, int r3, int col, uint16_t* out) {
    __shared__ __align__(1024) unsigned char buf[8 * 128 * 2];
    __shared__ __align__(8) uint64_t bar;
    const uint32_t sb = (uint32_t)__cvta_generic_to_shared(buf);
    const uint32_t mb = (uint32_t)__cvta_generic_to_shared(&bar);
    if (threadIdx.x == 0) {
        asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(mb));
        asm volatile("fence.mbarrier_init.release.cluster;");
        asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(mb), "r"(1024));
        asm volatile("cp.async.bulk.tensor.2d.shared::cluster.global.tile::gather4.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4, %5, %6}], [%7];"
                     ::"r"(sb), "l"(&tm), "r"(col), "r"(r0), "r"(r1), "r"(r2), "r"(r3), "r"(mb) : "memory");
        asm volatile("cp.async.bulk.tensor.2d.shared::cluster.global.tile::gather4.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4, %5, %6}], [%7];"
                     ::"r"(sb + 512), "l"(&tm), "r"(col), "r"(r0 + 10), "r"(r1 + 10), "r"(r2 + 10), "r"(r3 + 10), "r"(mb) : "memory");
        asm volatile("{\n.reg .pred p;\nW: mbarrier.try_wait.parity.shared::cta.b64 p, [%0], 0;\n@!p bra W;\n}" ::"r"(mb));
    }
    __syncthreads();
    for (int i = threadIdx.x; i < 512; i += blockDim.x) out[i] = reinterpret_cast<uint16_t*>(buf)[i];
}

int main() {
    const int rows = 1000, cols = 384;
    std::vector<uint16_t> h(rows * cols);
    for (int r = 0; r < rows; ++r)
        for (int c = 0; c < cols; ++c) h[r * cols + c] = (uint16_t)(r * 64 + (c >> 3));   // encodes (row, 16-byte chunk)
    uint16_t *d, *o;
    cudaMalloc(&d, h.size() * 2);
    cudaMalloc(&o, 1024);
    cudaMemcpy(d, h.data(), h.size() * 2, cudaMemcpyHostToDevice);
    void* fn = nullptr;
    cudaDriverEntryPointQueryResult q;
    cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fn, cudaEnableDefault, &q);
    auto enc = (CUresult(*)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*, const cuuint64_t*,
                            const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave, CUtensorMapSwizzle,
                            CUtensorMapL2promotion, CUtensorMapFloatOOBfill))fn;
    for (int bh : {1}) {
        CUtensorMap tm;
        cuuint64_t dims[2] = {(cuuint64_t)cols, (cuuint64_t)rows};
        cuuint64_t strides[1] = {(cuuint64_t)cols * 2};
        cuuint32_t box[2] = {64, (cuuint32_t)bh};
        cuuint32_t es[2] = {1, 1};
        CUresult rc = enc(&tm, CU_TENSOR_MAP_DATA_TYPE_FLOAT16, 2, d, dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                          CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
        printf("box height %d: encode rc %d\n", bh, (int)rc);
        if (rc) continue;
        cudaMemset(o, 0xff, 1024);
        k<<<1, 128>>>(tm, 7, 500, 3, 999, 128, o);
        cudaError_t e = cudaDeviceSynchronize();
        printf("  kernel: %s\n", cudaGetErrorString(e));
        if (e) return 1;
        std::vector<uint16_t> r(512);
        cudaMemcpy(r.data(), o, 1024, cudaMemcpyDeviceToHost);
        for (int row = 0; row < 8; ++row) {
            printf("  smem row %d:", row);
            for (int ch = 0; ch < 8; ++ch) {
                const uint16_t v = r[row * 64 + ch * 8];
                printf(" (r%d c%d)", v / 64, v % 64);
            }
            printf("\n");
        }
    }
    return 0;
}
