// tables.cu -- a4 for L > 1 hash tables ("L hash tables are used and
// each of them is constructed independently with different dim-M hash
// functions"; A(v) = every point in the query's buckets, deduplicated across
// tables -- reading R24).
//
// The rows of X are stored once, in table-0 order (every bucket of table 0 is
// a contiguous slab); table l's buckets are runs of table-l positions mapped
// to table-0 positions by pos_l.  Every table sorts by leaf first, so all
// candidates of a query lie inside its leaf's table-0 range [leaf_pos[g],
// leaf_pos[g+1]).  One CTA per query marks them in a bitmap of the leaf's rows
// held in shared memory (1 bit per row: 19.5 KB for a 156 K-row leaf), then
// compacts the set bits in ascending order: the deduplicated candidate list,
// sorted by table-0 position (= bucket order, good locality for the
// short-list).  Work per query: sum of the L tables' |A0_l(q)| bit sets (4-byte
// pos reads for l > 0) + one pass over the leaf's bitmap words.
#include "internal.cuh"
#include "query_kernels.cuh"

namespace blsh {

namespace {

constexpr int kUT = 512;

__global__ void k_raw_counts(UnionArgs u) {
    const int64_t q = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (q >= u.nq) return;
    int64_t r = 0;
    for (int l = 0; l < u.L; ++l) r += u.cnt[l][q];
    if (u.hrows) r += u.hrows[q];
    u.raw[q] = r;
}

__global__ void __launch_bounds__(kUT) k_union_tables(UnionArgs u) {
    extern __shared__ uint32_t bm[];
    __shared__ uint32_t wsum[kUT / 32];
    __shared__ int64_t s_base;
    const int64_t q = blockIdx.x;
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    if (u.qoor[q] & 2) {   // leaf owned by another shard
        if (tid == 0) u.out_cnt[q] = 0;
        return;
    }
    const int g = u.qleaf[q];
    const int64_t lb = u.leaf_pos[g];
    const int64_t rows = u.leaf_pos[g + 1] - lb;
    const int nw = (int)((rows + 31) >> 5);
    for (int i = tid; i < nw; i += kUT) bm[i] = 0u;
    __syncthreads();
    for (int l = 0; l < u.L; ++l) {
        const uint2* iv = u.ivl[l] + (size_t)q * (u.T + 1);
        const uint32_t* pos = u.pos[l];
        for (int p = 0; p <= u.T; ++p) {
            const uint2 r = iv[p];
            for (int64_t j = (int64_t)r.x + tid; j < (int64_t)r.y; j += kUT) {
                const int64_t x = (pos ? (int64_t)__ldg(pos + j) : j) - lb;
                atomicOr(&bm[x >> 5], 1u << (x & 31));
            }
        }
    }
    if (u.hlevel && u.he[q] > u.hs[q]) {   // E8 hierarchy node: its buckets' rows
        const int lv = u.hlevel[q];
        const uint32_t* bu = (lv >= 1 && lv <= kE8Levels) ? u.lv_bu[lv] : nullptr;
        for (int64_t b = u.hs[q] + tid; b < u.he[q]; b += kUT) {
            const uint32_t bk = bu ? bu[b] : (uint32_t)b;
            for (int64_t j = u.uoff[bk]; j < (int64_t)u.uoff[bk + 1]; ++j) {
                const int64_t x = j - lb;
                atomicOr(&bm[x >> 5], 1u << (x & 31));
            }
        }
    }
    __syncthreads();
    // ordered compaction: block-wide exclusive scan of the word popcounts
    uint32_t* out = u.list + u.raw_off[q];
    if (tid == 0) s_base = 0;
    __syncthreads();
    for (int w0 = 0; w0 < nw; w0 += kUT) {
        const int w = w0 + tid;
        const uint32_t bits = w < nw ? bm[w] : 0u;
        const int pc = __popc(bits);
        int incl = pc;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const int t = __shfl_up_sync(BLSH_FULL, incl, o);
            if (lane >= o) incl += t;
        }
        if (lane == 31) wsum[warp] = (uint32_t)incl;
        __syncthreads();
        if (warp == 0) {
            int v = lane < kUT / 32 ? (int)wsum[lane] : 0;
            int vi = v;
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                const int t = __shfl_up_sync(BLSH_FULL, vi, o);
                if (lane >= o) vi += t;
            }
            if (lane < kUT / 32) wsum[lane] = (uint32_t)(vi - v);   // exclusive warp offsets
        }
        __syncthreads();
        int64_t o = s_base + wsum[warp] + (incl - pc);
        uint32_t b = bits;
        while (b) {
            const int t = __ffs(b) - 1;
            out[o++] = (uint32_t)(lb + ((int64_t)w << 5) + t);
            b &= b - 1;
        }
        __syncthreads();
        if (tid == kUT - 1) s_base = o;   // the last thread's end is the chunk total
        __syncthreads();
    }
    if (tid == 0) u.out_cnt[q] = s_base;
}

}  // namespace

void launch_raw_counts(const UnionArgs& u, cudaStream_t s) {
    if (u.nq == 0) return;
    k_raw_counts<<<(unsigned)((u.nq + 255) / 256), 256, 0, s>>>(u);
    BLSH_LAUNCH_CHECK();
}

void launch_union_tables(const UnionArgs& u, int64_t max_leaf_rows, cudaStream_t s) {
    if (u.nq == 0) return;
    const size_t smem = (size_t)((max_leaf_rows + 31) / 32) * 4 + 16;
    if (smem > 200 * 1024) throw Error(BLSH_ERR_UNSUPPORTED, "L > 1 needs leaves of <= 1,600,000 points (increase n_leaves)");
    BLSH_CUDA(cudaFuncSetAttribute(k_union_tables, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    k_union_tables<<<(unsigned)u.nq, kUT, smem, s>>>(u);
    BLSH_LAUNCH_CHECK();
}

}  // namespace blsh
