// tiled_kernel.cuh -- the query-tiled short-list kernel (included by
// shortlist_tiled.cu inside its anonymous namespace).
//
// Warp specialisation: warps 0-7 score, warp 8 is the TMA producer.  The
// producer streams the item's rows of the tile's candidate union through a
// 3-stage ring of 32-row buffers: per stage, one lane per row finds the row's
// segment (binary search on the segment prefix), writes (row, query-mask) into
// the stage's metadata, and issues a 1-D bulk copy (cp.async.bulk) of the row
// into a 16-byte padded slot; completion is tracked by the stage's `full`
// mbarrier (expect_tx), reuse by its `empty` mbarrier (one arrival per scoring
// warp).  No CTA-wide barrier inside the loop, so scoring warps drift freely
// within the ring.  Scoring warp w owns tile queries 4w..4w+3; per stage each
// lane scores its row against the subset of those queries that some lane of
// the warp needs (compile-time query subsets, 15 variants).

constexpr int kStages = 3;
constexpr int kScorers = 8;                   // scoring warps
constexpr int kTiledThreads = (kScorers + 1) * 32;

__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}

// d^2 of this lane's row against the queries in QM (bit j = query j of the
// warp), fp32 direct form; partial sums of <= 64 terms (two 32-term
// accumulators per block of 16 float4), blocks summed in order (R22).
template <int QM>
__device__ __forceinline__ void score_rows(const float4* __restrict__ xr, const float4* __restrict__ q4, int nv4,
                                           float* tot) {
#pragma unroll
    for (int j = 0; j < 4; ++j) tot[j] = 0.f;
    for (int vb = 0; vb < nv4; vb += 16) {
        const int ve = min(nv4, vb + 16);
        float a0[4] = {0.f, 0.f, 0.f, 0.f}, a1[4] = {0.f, 0.f, 0.f, 0.f};
#pragma unroll 4
        for (int v = vb; v < ve; ++v) {
            const float4 x = xr[v];
#pragma unroll
            for (int j = 0; j < 4; ++j) {
                if (!((QM >> j) & 1)) continue;
                const float4 q = q4[j * nv4 + v];
                const float dx = q.x - x.x, dy = q.y - x.y, dz = q.z - x.z, dw = q.w - x.w;
                a0[j] = fmaf(dx, dx, a0[j]);
                a1[j] = fmaf(dy, dy, a1[j]);
                a0[j] = fmaf(dz, dz, a0[j]);
                a1[j] = fmaf(dw, dw, a1[j]);
            }
        }
#pragma unroll
        for (int j = 0; j < 4; ++j)
            if ((QM >> j) & 1) tot[j] += a0[j] + a1[j];
    }
}

__global__ void __launch_bounds__(kTiledThreads, 1) k_shortlist_tiled(TiledArgs a) {
    extern __shared__ __align__(128) unsigned char smraw[];
    uint64_t* full = reinterpret_cast<uint64_t*>(smraw);        // [kStages]
    uint64_t* empty = full + kStages;                           // [kStages]
    uint32_t* rmask = reinterpret_cast<uint32_t*>(smraw + 128); // [kStages][32]
    uint32_t* rid = rmask + kStages * 32;                       // [kStages][32]
    float* qs = reinterpret_cast<float*>(smraw + 1024);         // [QT][ds]
    const int ds = a.ds, nv4 = ds >> 2, pitch = ds + 4;
    float* rws = qs + (size_t)QT * ds;                          // [kStages][32][pitch]
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const int64_t item = blockIdx.x;
    int64_t r0, r1;
    const int64_t tile = item_tile_rows(a, item, &r0, &r1);
    const int nst = (int)((r1 - r0 + 31) / 32);
    for (int i = threadIdx.x; i < QT * nv4; i += kTiledThreads) {
        const int slot = i / nv4, v = i % nv4;
        const int64_t qp = a.tile_off[tile] + slot;
        float4 x = make_float4(0.f, 0.f, 0.f, 0.f);
        if (qp < a.tile_off[tile + 1]) x = reinterpret_cast<const float4*>(a.Q + (size_t)a.qorder[qp] * ds)[v];
        reinterpret_cast<float4*>(qs)[(size_t)slot * nv4 + v] = x;
    }
    if (threadIdx.x == 0) {
        for (int s = 0; s < kStages; ++s) {
            mbar_init(&full[s], 1);
            mbar_init(&empty[s], kScorers);
        }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    const uint32_t rowbytes = (uint32_t)ds * 4u;
    if (warp == kScorers) {
        // ---------------- producer ----------------
        const Seg* S = a.segs + (size_t)tile * a.segcap;
        const int ns = a.nseg[tile];
        int cs = 0;   // segment containing the first row of the current stage
        {
            int l2 = 0, h2 = ns;   // last segment with off <= r0 (once per item)
            while (h2 - l2 > 1) {
                const int m = (l2 + h2) >> 1;
                if ((int64_t)S[m].off <= r0) l2 = m;
                else h2 = m;
            }
            cs = l2;
        }
        Seg sgn = (cs + lane < ns) ? S[cs + lane] : Seg{0u, 0u, 0u, 0xFFFFFFFFu};
        for (int j = 0; j < nst; ++j) {
            const int b = j % kStages;
            const int64_t rs = r0 + 32 * (int64_t)j;
            const uint32_t r = (uint32_t)(rs + lane);
            const bool v = (int64_t)r < r1;
            const int64_t left = r1 - rs;
            const int n = left < 32 ? (int)left : 32;
            // the 32 rows of a stage lie in at most 32 consecutive segments starting at cs
            const Seg sgl = sgn;
            int my = 0;
#pragma unroll 8
            for (int t = 0; t < 32; ++t) {
                const uint32_t rt = __shfl_sync(BLSH_FULL, r, t);
                const unsigned bm = __ballot_sync(BLSH_FULL, sgl.off <= rt);
                if (lane == t) my = __popc(bm) - 1;
            }
            const uint32_t s_start = __shfl_sync(BLSH_FULL, sgl.start, my);
            const uint32_t s_off = __shfl_sync(BLSH_FULL, sgl.off, my);
            const uint32_t s_mask = __shfl_sync(BLSH_FULL, sgl.mask, my);
            const uint32_t row = s_start + (r - s_off);
            const uint32_t msk = v ? s_mask : 0u;
            cs += __popc(__ballot_sync(BLSH_FULL, sgl.off <= (uint32_t)(rs + 32))) - 1;
            if (j + 1 < nst) sgn = (cs + lane < ns) ? S[cs + lane] : Seg{0u, 0u, 0u, 0xFFFFFFFFu};   // prefetch
            if (j >= kStages) mbar_wait(&empty[b], (uint32_t)((j / kStages - 1) & 1));
            rmask[b * 32 + lane] = msk;
            rid[b * 32 + lane] = row;
            __syncwarp();
            if (lane == 0) {
                asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
                mbar_expect_tx(&full[b], (uint32_t)n * rowbytes);
            }
            __syncwarp();
            if (v) bulk_g2s(rws + (size_t)(b * 32 + lane) * pitch, a.Xp + (size_t)row * ds, rowbytes, &full[b]);
        }
        return;
    }
    // ---------------- scorers ----------------
    TopK tk[4];
    unsigned long long thr[4];
#pragma unroll
    for (int j = 0; j < 4; ++j) { tk[j] = TopK{kEmpty, kEmpty}; thr[j] = kEmpty; }
    const int k = a.k;
    unsigned long long evaluated = 0ull;
    const float4* q4 = reinterpret_cast<const float4*>(qs) + (size_t)(warp * 4) * nv4;
    for (int j = 0; j < nst; ++j) {
        const int b = j % kStages;
        mbar_wait(&full[b], (uint32_t)((j / kStages) & 1));
        const int64_t left = r1 - (r0 + 32 * (int64_t)j);
        const bool valid = lane < left;
        const uint32_t msk = valid ? rmask[b * 32 + lane] : 0u;
        const uint32_t prow = rid[b * 32 + lane];
        const uint32_t myq = (msk >> (warp * 4)) & 15u;
        unsigned needq = 0;
#pragma unroll
        for (int q = 0; q < 4; ++q)
            if (__ballot_sync(BLSH_FULL, (myq >> q) & 1u)) needq |= 1u << q;
        if (needq) {
            evaluated += 32ull * (unsigned long long)__popc(needq);
            const uint32_t id = valid ? __ldg(a.perm + prow) : 0u;   // used after scoring
            const float4* xr = reinterpret_cast<const float4*>(rws + (size_t)(b * 32 + lane) * pitch);
            float tot[4];
            switch (needq) {
#define BLSH_SCORE_CASE(QMV) case QMV: score_rows<QMV>(xr, q4, nv4, tot); break;
                BLSH_SCORE_CASE(1) BLSH_SCORE_CASE(2) BLSH_SCORE_CASE(3) BLSH_SCORE_CASE(4)
                BLSH_SCORE_CASE(5) BLSH_SCORE_CASE(6) BLSH_SCORE_CASE(7) BLSH_SCORE_CASE(8)
                BLSH_SCORE_CASE(9) BLSH_SCORE_CASE(10) BLSH_SCORE_CASE(11) BLSH_SCORE_CASE(12)
                BLSH_SCORE_CASE(13) BLSH_SCORE_CASE(14) BLSH_SCORE_CASE(15)
#undef BLSH_SCORE_CASE
                default: break;
            }
            __syncwarp();
            if (lane == 0) mbar_arrive(&empty[b]);   // row data consumed; metadata already in registers
#pragma unroll
            for (int q = 0; q < 4; ++q) {
                if (!((needq >> q) & 1u)) continue;
                const bool mine = (myq >> q) & 1u;
                const unsigned long long key = mine ? pack_entry(tot[q], id) : kEmpty;
                topk_offer(tk[q], thr[q], key, k, lane);
            }
        } else {
            __syncwarp();
            if (lane == 0) mbar_arrive(&empty[b]);
        }
    }
#pragma unroll
    for (int q = 0; q < 4; ++q) {
        if (q == 0 && lane == 0 && a.counters) atomicAdd(a.counters, evaluated);
        unsigned long long* out = a.partials + ((size_t)item * QT + warp * 4 + q) * k;
        if (lane < k) out[lane] = tk[q].e0;
        if (lane + 32 < k) out[lane + 32] = tk[q].e1;
    }
}
