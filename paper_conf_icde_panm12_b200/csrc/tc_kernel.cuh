// tc_kernel.cuh -- query-tiled short-list with a tensor-core screen
// (included by shortlist_tiled.cu inside its anonymous namespace).
//
// For a tile of <= QT = 32 queries and a 128-row block of the tile's candidate
// union, the 128 x 32 dot products of the CENTRED vectors (x - c)(q - c),
// c = mean of the tile's queries, are one tcgen05.mma chain (kind::tf32,
// M = 128, N = 32, K = d in steps of 8) accumulated in TMEM.  The epilogue
// turns them into approximate distances ~d2 = |q'|^2 + |x'|^2 - 2 q'.x' with
// the bound |~d2 - d2| <= m = 4e-3 (|q'|^2 + |x'|^2) + 1e-5 ~d2 (TF32 operand
// truncation + fp32 accumulation, with margin).  U_j, the k-th smallest
// ~d2 + m seen for query j, bounds its exact k-th distance from above, so a
// pair with ~d2 - m > U_j can never enter the top-k.  Pairs that pass are
// buffered (lower bound, row) and, after the whole union has been streamed,
// only those with lower bound <= the final U_j are rescored EXACTLY in the
// fp32 direct form of k_shortlist (R22).  The tensor cores only decide which
// pairs need exact work; results equal the SIMT kernels' up to rounding of the
// direct form (identical to k_shortlist's).
//
// Warp roles (13 warps):
//   0-7  converters: per block, find each row's table position and query mask
//        in the tile's segment list, gather the rows from HBM (coalesced
//        16-byte loads: 8 rows x 64 bytes per instruction, the next chunk's
//        loads in flight while the current one is converted), subtract c,
//        write the TF32 A operand in the K-major no-swizzle UMMA layout
//        (8-row x 16-byte core matrices), |x'|^2 per row;
//   8    MMA issuer (one elected lane) + TMEM allocation;
//   9-12 epilogue: tcgen05.ld of the 32 accumulators of its 32 rows, transpose
//        through shared memory so that lane j screens query j: per-lane sorted
//        upper-bound lists and per-lane pair buffers (registers and lane-private
//        memory: no atomics or locks on the hot path), final exact rescoring.
// Pipelines: 4-slot ring of 64-column A chunks (full / empty mbarriers; the
// MMA frees a slot with tcgen05.commit), 4 TMEM accumulator slots and 4
// row-metadata slots (tmem_full by commit, tmem_empty / meta_free by the
// epilogue).

constexpr int kTcRows = 128;               // M
constexpr int kTcChunk = 64;               // K columns per A chunk
constexpr int kTcSlots = 4;                // A chunk ring
constexpr int kTcAhead = 3;                // staged chunks in flight ahead of the conversion (< kTcSlots)
constexpr int kTcBlk = 4;                  // TMEM / metadata slots
#ifndef BLSH_TC_Q
#define BLSH_TC_Q 2
#endif
constexpr int kTcQ = BLSH_TC_Q;            // column parts of a 64-column chunk (one converter warp each per quadrant)
constexpr int kTcCols = 64 / kTcQ;         // columns per converter warp and chunk (32 or 16)
constexpr int kTcPieces = kTcCols / 4;     // 16-byte pieces per staged row
constexpr int kTcConv = 4 * kTcQ;          // converter warps
constexpr int kTcMmaWarp = kTcConv;
constexpr int kTcEpi0 = kTcConv + 1;       // first epilogue warp
constexpr int kTcThreads = (kTcConv + 5) * 32;
constexpr int kTcMaxK = 32;                // k supported by the TC path
constexpr int kTcScap = 96;                // buffered pairs per (item, query, epilogue warp)
constexpr uint32_t kTcStageBytes = kTcRows * kTcChunk * 4;   // 32 KB staging per chunk
constexpr uint32_t kTcChunkBytes = kTcStageBytes;
constexpr int kTcASlots = 4;               // A ring in tensor memory (64 columns each)
constexpr uint32_t kTcACol0 = kTcBlk * 32; // first TMEM column of the A ring (after the accumulators)
// instruction descriptor: D f32, A/B tf32, K-major both, N = 32, M = 128
constexpr uint32_t kTcIdesc = (1u << 4) | (2u << 7) | (2u << 10) | ((32u >> 3) << 17) | ((128u >> 4) << 24);

__device__ __forceinline__ uint64_t umma_desc(uint32_t saddr, uint32_t lbo, uint32_t sbo) {
    uint64_t d = 0;
    d |= (uint64_t)((saddr >> 4) & 0x3FFFu);
    d |= (uint64_t)((lbo >> 4) & 0x3FFFu) << 16;
    d |= (uint64_t)((sbo >> 4) & 0x3FFFu) << 32;
    d |= 1ull << 46;   // descriptor version for sm_100
    return d;          // base offset 0, SWIZZLE_NONE
}
__device__ __forceinline__ void tc_mma(uint32_t d_tmem, uint64_t adesc, uint64_t bdesc, uint32_t accum) {
    asm volatile(
        "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
        "tcgen05.mma.cta_group::1.kind::tf32 [%0], %1, %2, %3, p;\n\t}" ::"r"(d_tmem),
        "l"(adesc), "l"(bdesc), "r"(kTcIdesc), "r"(accum)
        : "memory");
}
// A from tensor memory (tf32, M = 128: row m in lane m, one K element per column)
__device__ __forceinline__ void tc_mma_ts(uint32_t d_tmem, uint32_t a_tmem, uint64_t bdesc, uint32_t accum) {
    asm volatile(
        "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
        "tcgen05.mma.cta_group::1.kind::tf32 [%0], [%1], %2, %3, p;\n\t}" ::"r"(d_tmem),
        "r"(a_tmem), "l"(bdesc), "r"(kTcIdesc), "r"(accum)
        : "memory");
}
__device__ __forceinline__ void tc_commit(uint64_t* bar) {
    asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(smem_u32(bar))
                 : "memory");
}
__device__ __forceinline__ void tc_fence_after() { asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void tc_fence_before() { asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void named_bar(int id, int n) { asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(n) : "memory"); }

__device__ __forceinline__ void tmem_st32(uint32_t taddr, const uint32_t* r) {
    asm volatile(
        "tcgen05.st.sync.aligned.32x32b.x32.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16,"
        "%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31,%32};" ::"r"(taddr),
        "r"(r[0]), "r"(r[1]), "r"(r[2]), "r"(r[3]), "r"(r[4]), "r"(r[5]), "r"(r[6]), "r"(r[7]),
        "r"(r[8]), "r"(r[9]), "r"(r[10]), "r"(r[11]), "r"(r[12]), "r"(r[13]), "r"(r[14]), "r"(r[15]),
        "r"(r[16]), "r"(r[17]), "r"(r[18]), "r"(r[19]), "r"(r[20]), "r"(r[21]), "r"(r[22]), "r"(r[23]),
        "r"(r[24]), "r"(r[25]), "r"(r[26]), "r"(r[27]), "r"(r[28]), "r"(r[29]), "r"(r[30]), "r"(r[31])
        : "memory");
    asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
}

__device__ __forceinline__ void tmem_st16(uint32_t taddr, const uint32_t* r) {
    asm volatile(
        "tcgen05.st.sync.aligned.32x32b.x16.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16};"
        ::"r"(taddr), "r"(r[0]), "r"(r[1]), "r"(r[2]), "r"(r[3]), "r"(r[4]), "r"(r[5]), "r"(r[6]), "r"(r[7]),
        "r"(r[8]), "r"(r[9]), "r"(r[10]), "r"(r[11]), "r"(r[12]), "r"(r[13]), "r"(r[14]), "r"(r[15])
        : "memory");
    asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
}

__device__ __forceinline__ void tmem_ld32(uint32_t taddr, float* v) {
    uint32_t r[32];
    asm volatile(
        "tcgen05.ld.sync.aligned.32x32b.x32.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,"
        "%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%32];"
        : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]),
          "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15]),
          "=r"(r[16]), "=r"(r[17]), "=r"(r[18]), "=r"(r[19]), "=r"(r[20]), "=r"(r[21]), "=r"(r[22]), "=r"(r[23]),
          "=r"(r[24]), "=r"(r[25]), "=r"(r[26]), "=r"(r[27]), "=r"(r[28]), "=r"(r[29]), "=r"(r[30]), "=r"(r[31])
        : "r"(taddr));
    asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
#pragma unroll
    for (int i = 0; i < 32; ++i) v[i] = __uint_as_float(r[i]);
}

struct TcSmem {
    uint64_t afull[kTcASlots], aempty[kTcASlots];
    uint64_t tfull[kTcBlk], tempty[kTcBlk], xready[kTcBlk], mfree[kTcBlk];
    uint32_t tmem_base;
    alignas(16) float qn[QT];                // |q'|^2
    uint32_t rpos[kTcBlk][kTcRows];          // table row of each block row
    uint32_t rmask[kTcBlk][kTcRows];         // query mask of each block row (0 = padding)
    float xn2[kTcBlk][kTcQ][kTcRows];        // |x'|^2, per column part
    alignas(16) uint32_t umin[QT];           // per query: smallest k-th upper bound over the epilogue warps (bits)
    int scnt[4][QT];                         // per (epilogue warp, query): buffered pairs
    alignas(16) float cen[512];              // centre of the tile (mean of its queries)
    float tr[4][32 * 33];                    // per epilogue warp: transposed dots [query][row], padded
    uint4 rinfo[4][32];                      // per epilogue warp: (|x'|^2 bits, query mask, table row) per row
};

__device__ __forceinline__ void tk_insert(unsigned long long* L, int k, unsigned long long key) {
    if (key < L[k - 1]) {
        int p = k - 1;
        while (p > 0 && L[p - 1] > key) { L[p] = L[p - 1]; --p; }
        L[p] = key;
    }
}

__device__ __forceinline__ void tc_stamp(const TiledArgs& a, int64_t item, int p) {
    if (a.tstamp) {
        unsigned long long t;
        asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
        a.tstamp[item * 16 + p] = t;
    }
}

// KT: length of the per-lane upper-bound lists (>= k; the first KT - k entries are -inf
// placeholders, so the k-th smallest real bound is always ulr[KT - 1]).
template <int KT>
__global__ void __launch_bounds__(kTcThreads, 1) k_shortlist_tc(TiledArgs a) {
    extern __shared__ __align__(1024) unsigned char smraw[];
    TcSmem& S = *reinterpret_cast<TcSmem*>(smraw);
    const int ds = a.ds, nv4 = ds >> 2, kp_total = ds >> 2;   // 16-byte K pieces
    unsigned char* opbase = smraw + ((sizeof(TcSmem) + 1023) & ~size_t(1023));
    unsigned char* Bop = opbase;                                    // [QT x ds] tf32, UMMA K-major
    unsigned char* Aop = Bop + (size_t)QT * ds * 4;                 // [kTcSlots] staging (8 warps x 32 rows x 128 B)
    float* Qf = reinterpret_cast<float*>(Aop);                      // setup only: original queries (aliases A)
    const uint32_t sboB = (uint32_t)kp_total * 128u;
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const int64_t item = blockIdx.x;
    int64_t r0, r1;
    const int64_t tile = item_tile_rows(a, item, &r0, &r1);
    const int nblk = (int)((r1 - r0 + kTcRows - 1) / kTcRows);
    const int nchunk = ds / kTcChunk;
    const int k = a.k;
    if (threadIdx.x == 0) tc_stamp(a, item, 0);
    // ---- setup: queries, centre c = mean of the tile's queries, B operand (q - c), |q'|^2 ----
    const int64_t q0 = a.tile_off[tile];
    const int nqt = (int)(a.tile_off[tile + 1] - q0);
    for (int i = threadIdx.x; i < QT * nv4; i += kTcThreads) {
        const int n = i / nv4, v = i % nv4;
        reinterpret_cast<float4*>(Qf)[i] = n < nqt ? reinterpret_cast<const float4*>(a.Q + (size_t)a.qorder[q0 + n] * ds)[v]
                                                   : make_float4(0.f, 0.f, 0.f, 0.f);
    }
    __syncthreads();
    for (int j = threadIdx.x; j < ds; j += kTcThreads) {
        float s = 0.f;
        for (int n = 0; n < nqt; ++n) s += Qf[(size_t)n * ds + j];
        S.cen[j] = s / (float)nqt;
    }
    __syncthreads();
    const float* cen = S.cen;
    for (int i = threadIdx.x; i < QT * kp_total; i += kTcThreads) {
        const int n = i % QT, kp = i / QT;
        float4 v = make_float4(0.f, 0.f, 0.f, 0.f);
        if (n < nqt) {
            const float4 x = reinterpret_cast<const float4*>(Qf + (size_t)n * ds)[kp];
            const float4 cc = reinterpret_cast<const float4*>(cen)[kp];
            v = make_float4(x.x - cc.x, x.y - cc.y, x.z - cc.z, x.w - cc.w);
        }
        *reinterpret_cast<float4*>(Bop + (size_t)(n >> 3) * sboB + (size_t)kp * 128 + (n & 7) * 16) = v;
    }
    for (int n = warp; n < QT; n += kTcThreads / 32) {   // |q'|^2: one warp per query
        float s = 0.f;
        if (n < nqt) {
            const float* qq = Qf + (size_t)n * ds;
            for (int j = lane; j < ds; j += 32) {
                const float e = qq[j] - cen[j];
                s = fmaf(e, e, s);
            }
        }
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(BLSH_FULL, s, o);
        if (lane == 0) {
            S.qn[n] = s;
        }
    }
    if (threadIdx.x < QT) S.umin[threadIdx.x] = 0x7F800000u;
    if (threadIdx.x == 0) {
        for (int s = 0; s < kTcASlots; ++s) {
            mbar_init(&S.afull[s], kTcConv);
            mbar_init(&S.aempty[s], 1);
        }
        for (int s = 0; s < kTcBlk; ++s) {
            mbar_init(&S.tfull[s], 1);
            mbar_init(&S.tempty[s], 4);
            mbar_init(&S.xready[s], kTcConv);
            mbar_init(&S.mfree[s], 4);
        }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    if (warp == kTcMmaWarp) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"(smem_u32(&S.tmem_base)));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");   // B operand visible to the tensor core
    tc_fence_before();
    __syncthreads();                                                // Qf (aliasing the A ring) is dead from here
    tc_fence_after();
    const uint32_t tbase = S.tmem_base;
    if (threadIdx.x == 0) tc_stamp(a, item, 1);

    if (warp < kTcConv) {
        // ======================= converters =======================
        // Converter warp w owns TMEM lane quadrant qd = w % 4 (block rows 32 qd + lane, one row
        // per lane) and half hf = w / 4 of every 64-column chunk.  Its 32 rows x 32 columns are
        // copied by 16-byte cp.async into a warp-private staging area (kTcAhead chunks ahead;
        // 16-byte pieces XOR-swizzled by row so both the copy and the row-per-lane reads are
        // bank-conflict free), then each lane subtracts c from its row, accumulates |x'|^2 and
        // writes the 32 TF32 operands to the A ring in tensor memory (tcgen05.st).  Staging is
        // warp-private (cp.async.wait_group orders it), so only the TMEM A slots and the block
        // metadata need cross-warp barriers.
        const int qd = warp & 3, hf = warp >> 2;   // quadrant, column part
        const int nch_total = nblk * nchunk;
        const uint4* RI = a.rowinfo + a.rows_off[tile];
        unsigned char* stg = Aop + (size_t)warp * (32 * kTcCols * 4);   // + slot * kTcStageBytes
        // 16-byte piece p of staged row r lives at r * kTcCols * 4 + ((p ^ swz(r)) << 4): conflict-free
        // for the copies and for the row-per-lane reads (8-lane phases see 8 distinct bank groups)
        auto swz = [](int r) { return kTcPieces == 8 ? (r & 7) : ((r >> 1) & 3); };
        auto fetch = [&](int b) {                          // this lane's row entry of block b
            const int64_t r = r0 + (int64_t)b * kTcRows + 32 * qd + lane;
            if (b < nblk && r < r1) { const uint4 f = RI[r]; return make_uint2(f.x, f.y); }
            return make_uint2(0u, 0u);
        };
        uint2 e_next = fetch(0), e_iss = make_uint2(0u, 0u);
        auto issue = [&](int g) {                          // cp.async of chunk g (this warp's part)
            if (g < nch_total) {
                const int b = g / nchunk, c = g - b * nchunk;
                if (c == 0) {                              // new block: its row metadata
                    const int ms = b & (kTcBlk - 1);
                    e_iss = e_next;
                    e_next = fetch(b + 1);
                    // every converter warp writes slot ms (metadata or |x'|^2): wait until the
                    // epilogue has released it
                    if (b >= kTcBlk) mbar_wait(&S.mfree[ms], (uint32_t)(((b / kTcBlk) - 1) & 1));
                    if (hf == 0) {
                        S.rpos[ms][32 * qd + lane] = e_iss.x;
                        S.rmask[ms][32 * qd + lane] = e_iss.y;
                    }
                }
                const uint32_t sb = smem_u32(stg + (size_t)(g % kTcSlots) * kTcStageBytes);
                const bool nol = (a.dbgmode & 2) != 0;
                const int p = lane % kTcPieces;
#pragma unroll
                for (int it = 0; it < kTcPieces; ++it) {   // 32 / kTcPieces rows per instruction
                    const int r = it * (32 / kTcPieces) + lane / kTcPieces;
                    const uint32_t pos = __shfl_sync(BLSH_FULL, e_iss.x, r);
                    const uint32_t msk = __shfl_sync(BLSH_FULL, e_iss.y, r);
                    const float* src = a.Xp + (size_t)pos * ds + c * kTcChunk + hf * kTcCols + p * 4;
                    const uint32_t dst = sb + (uint32_t)(r * kTcCols * 4 + ((p ^ swz(r)) << 4));
                    asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;" ::"r"(dst), "l"(src),
                                 "r"((msk != 0u && !nol) ? 16u : 0u)
                                 : "memory");
                }
            }
            asm volatile("cp.async.commit_group;" ::: "memory");   // (possibly empty: uniform group count)
        };
        for (int g = 0; g < kTcAhead; ++g) issue(g);
        float xs = 0.f;
        const uint32_t tl = (uint32_t)(32 * qd) << 16;   // TMEM lane base of this warp
        for (int g = 0; g < nch_total; ++g) {
            issue(g + kTcAhead);
            asm volatile("cp.async.wait_group %0;" ::"n"(kTcAhead) : "memory");   // chunk g has landed
            const int b = g / nchunk, c = g - b * nchunk;
            const int slot = g % kTcSlots;
            const unsigned char* row = stg + (size_t)slot * kTcStageBytes + lane * (kTcCols * 4);
            uint32_t v[kTcCols];
#pragma unroll
            for (int p = 0; p < kTcPieces; ++p) {
                float4 x = *reinterpret_cast<const float4*>(row + ((p ^ swz(lane)) << 4));
                const float4 cc = reinterpret_cast<const float4*>(cen)[(c * kTcChunk + hf * kTcCols) / 4 + p];
                x.x -= cc.x; x.y -= cc.y; x.z -= cc.z; x.w -= cc.w;
                xs = fmaf(x.x, x.x, xs);
                xs = fmaf(x.y, x.y, xs);
                xs = fmaf(x.z, x.z, xs);
                xs = fmaf(x.w, x.w, xs);
                v[4 * p] = __float_as_uint(x.x);
                v[4 * p + 1] = __float_as_uint(x.y);
                v[4 * p + 2] = __float_as_uint(x.z);
                v[4 * p + 3] = __float_as_uint(x.w);
            }
            const int as = g % kTcASlots;
            if (g >= kTcASlots) mbar_wait(&S.aempty[as], (uint32_t)((g / kTcASlots - 1) & 1));
            tc_fence_after();
            if (kTcCols == 32) tmem_st32(tbase + tl + kTcACol0 + (uint32_t)(as * kTcChunk + hf * kTcCols), v);
            else tmem_st16(tbase + tl + kTcACol0 + (uint32_t)(as * kTcChunk + hf * kTcCols), v);
            tc_fence_before();
            __syncwarp();
            if (lane == 0) mbar_arrive(&S.afull[as]);
            if (c == nchunk - 1) {
                const int ms = b & (kTcBlk - 1);
                S.xn2[ms][hf][32 * qd + lane] = xs;
                xs = 0.f;
                __syncwarp();
                if (lane == 0) mbar_arrive(&S.xready[ms]);
            }
        }
        if (threadIdx.x == 0) tc_stamp(a, item, 2);
    } else if (warp == kTcMmaWarp) {
        // ======================= MMA issuer =======================
        for (int b = 0; b < nblk; ++b) {
            const int ts = b & (kTcBlk - 1);
            if (b >= kTcBlk) mbar_wait(&S.tempty[ts], (uint32_t)(((b / kTcBlk) - 1) & 1));
            tc_fence_after();
            const uint32_t dt = tbase + (uint32_t)ts * 32u;
            for (int c = 0; c < nchunk; ++c) {
                const int gch = b * nchunk + c;
                const int as = gch % kTcASlots;
                mbar_wait(&S.afull[as], (uint32_t)((gch / kTcASlots) & 1));
                tc_fence_after();
                if (lane == 0) {
                    const uint32_t at = tbase + kTcACol0 + (uint32_t)(as * kTcChunk);
                    const uint32_t bbase = smem_u32(Bop) + (uint32_t)(c * 16) * 128u;
#pragma unroll
                    for (int s = 0; s < kTcChunk / 8; ++s) {
                        const uint64_t bd = umma_desc(bbase + (uint32_t)s * 256u, 128u, sboB);
                        if (!(a.dbgmode & 4)) tc_mma_ts(dt, at + (uint32_t)s * 8u, bd, (c > 0 || s > 0) ? 1u : 0u);
                    }
                    tc_commit(&S.aempty[as]);
                    if (c == nchunk - 1) tc_commit(&S.tfull[ts]);
                }
                __syncwarp();
            }
        }
        if (lane == 0) tc_stamp(a, item, 3);
    } else {
        // ======================= epilogue =======================
        // Lane = row when the accumulators come out of TMEM (tcgen05.ld 32x32b), lane = query
        // for the screen: the 32 x 32 block of dot products is transposed through a padded
        // shared tile (conflict-free both ways), then lane j runs query j's screen over the
        // warp's 32 rows with its own sorted upper-bound list and its own pair buffer.  The
        // 32 lists are updated in parallel (no serial per-pair insertion, no ballots).
        const int ew = warp - kTcEpi0;          // 0..3
        const int quad = warp & 3;              // TMEM lane quadrant of this warp
        const int brow = quad * 32 + lane;      // block row of this lane (row phase)
        const int j = lane;                     // query of this lane (screen phase)
        // Screen bounds.  With s = |q'|^2 + |x'|^2 and t the TF32 dot of the centred vectors,
        // |(s - 2t) - d2| <= 2.03e-3 s (TF32 operands: 2^-10 relative each; fp32 sums), and
        // |s - 2t| <= 2.004 s, so lo = s (1 - kScr) - 2t <= d2 <= s (1 + kScr) - 2t = up with
        // kScr = 4.03e-3 (2x slack; the rounding of these few fp32 operations is ~1e-7 s).
        constexpr float kScr = 4.03e-3f;
        const float qn = S.qn[j];
        const float qa = qn * (1.0f - kScr), qb = qn * (1.0f + kScr);
        float ulr[KT];                          // sorted k smallest upper bounds of query j seen by this warp
#pragma unroll
        for (int p = 0; p < KT; ++p) ulr[p] = p < KT - k ? __int_as_float(0xFF800000) : __int_as_float(0x7F800000);
        int my_cnt = 0;                         // buffered pairs of query j in this warp's buffer
        bool my_fail = false;                   // buffer overflowed: k_tc_rescore scans all of j's rows exactly
        unsigned long long* SBj = a.sbuf + (((size_t)item * QT + j) * 4 + ew) * kTcScap;
        float* Tt = S.tr[ew];
        const bool screen = !(a.dbgmode & 1);
        for (int b = 0; b < nblk; ++b) {
            const int ts = b & (kTcBlk - 1);
            mbar_wait(&S.tfull[ts], (uint32_t)((b / kTcBlk) & 1));
            mbar_wait(&S.xready[ts], (uint32_t)((b / kTcBlk) & 1));
            tc_fence_after();
            float dot[32];
            tmem_ld32(tbase + ((uint32_t)(quad * 32) << 16) + (uint32_t)ts * 32u, dot);
            tc_fence_before();
            const uint32_t msk = S.rmask[ts][brow];
            float xn = S.xn2[ts][0][brow];
#pragma unroll
            for (int h = 1; h < kTcQ; ++h) xn += S.xn2[ts][h][brow];
            const uint32_t prow = S.rpos[ts][brow];
            __syncwarp();
            if (lane == 0) {
                mbar_arrive(&S.tempty[ts]);
                mbar_arrive(&S.mfree[ts]);
            }
            if (a.dbg && item == 0 && b == 0) {
                for (int jj = 0; jj < 32; ++jj) a.dbg[brow * 32 + jj] = dot[jj];
                a.dbg[4096 + brow] = xn;
                a.dbg[4096 + 128 + brow] = __uint_as_float(prow);
                a.dbg[4096 + 256 + brow] = __uint_as_float(msk);
                if (brow < 32) a.dbg[4096 + 384 + brow] = S.qn[brow];
            }
            if (!screen) continue;
            // transpose: row lane writes its 32 dots, column j -> Tt[j][lane]
#pragma unroll
            for (int jj = 0; jj < 32; ++jj) Tt[jj * 33 + lane] = dot[jj];
            S.rinfo[ew][lane] = make_uint4(__float_as_uint(xn * (1.0f - kScr)), __float_as_uint(xn * (1.0f + kScr)),
                                           msk, prow);
            __syncwarp();
            const float kth0 = ulr[KT - 1];
            float U = fminf(kth0, __uint_as_float(S.umin[j]));    // any warp's bound is valid
#pragma unroll 8
            for (int i = 0; i < 32; ++i) {
                const uint4 ri = S.rinfo[ew][i];                   // broadcast
                const float t2 = -2.0f * Tt[j * 33 + i];
                const float lo = (qa + __uint_as_float(ri.x)) + t2;
                if (((ri.z >> j) & 1u) && lo <= U && !my_fail) {   // rare: keep the pair (failed: nothing to keep)
                    const float up = (qb + __uint_as_float(ri.y)) + t2;
                    if (up < U) {                                  // sorted insert; only bounds below U matter
#pragma unroll
                        for (int p = KT - 1; p > 0; --p) ulr[p] = fmaxf(ulr[p - 1], fminf(ulr[p], up));
                        ulr[0] = fminf(ulr[0], up);
                        U = fminf(U, ulr[KT - 1]);
                    }
                    const unsigned long long e = ((unsigned long long)__float_as_uint(fmaxf(lo, 0.f)) << 32) | ri.w;
                    if (my_cnt == kTcScap) {                       // full: drop what the tighter U excludes
                        int c2 = 0;
                        for (int t = 0; t < kTcScap; ++t) {
                            const unsigned long long f = SBj[t];
                            if (__uint_as_float((uint32_t)(f >> 32)) <= U) SBj[c2++] = f;
                        }
                        my_cnt = c2;
                        // compaction freed < 1/4: the screen cannot separate this query's candidates
                        // (further compactions would rescan the buffer per pair) -> exact scan later
                        if (my_cnt > 3 * kTcScap / 4) my_fail = true;
                    }
                    if (!my_fail) SBj[my_cnt++] = e;
                }
            }
            if (ulr[KT - 1] < kth0) atomicMin(&S.umin[j], __float_as_uint(ulr[KT - 1]));
            __syncwarp();                                          // Tt / rinfo reused by the next block
        }
        S.scnt[ew][j] = my_fail ? -1 : my_cnt;
        if (a.counters && my_cnt) atomicAdd(a.counters, (unsigned long long)my_cnt);   // kept pairs
        if (warp == kTcEpi0 && lane == 0) tc_stamp(a, item, 4);
    }
    tc_fence_before();
    __syncthreads();
    if (warp == kTcMmaWarp) {
        tc_fence_after();
        asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" ::"r"(tbase));
    }
    if (threadIdx.x == 0) tc_stamp(a, item, 5);
    // ---- hand-off to k_tc_rescore: final bound U_j, buffered pair counts, overflow top-k ----
    if (threadIdx.x < QT) {
        const int j = threadIdx.x;
        a.ufin[(size_t)item * QT + j] = j < nqt ? S.umin[j] : 0u;   // 0.0f: nothing to rescore for padding slots
#pragma unroll
        for (int w = 0; w < 4; ++w)   // -1: this warp's buffer for j overflowed (full exact scan of j's rows)
            a.scnt[((size_t)item * QT + j) * 4 + w] = j < nqt ? min(S.scnt[w][j], kTcScap) : 0;
    }
}

// Exact rescoring of the TC screen's survivors, at full occupancy (one warp per
// (item, query)): the buffered pairs whose lower bound is <= the final U_j get the
// fp32 direct-form distance of k_shortlist (lane l: float4 columns l, l+32, ..,
// per-lane fmaf chain, butterfly; bit-identical to the warp short-list), four rows
// at a time, and a warp top-k.  A query whose pair buffer overflowed in the screen (its
// candidates are too close together for the TF32 bound to separate them) gets the exact
// distance to every row of the item that its query mask selects instead.
template <int NV>
__global__ void __launch_bounds__(256) k_tc_rescore(TiledArgs a) {
    const int lane = threadIdx.x & 31;
    const int64_t unit = blockIdx.x * (int64_t)8 + (threadIdx.x >> 5);
    if (unit >= a.n_items * QT) return;
    const int64_t item = unit / QT;
    const int j = (int)(unit % QT);
    int64_t r0, r1;
    const int64_t lo = item_tile_rows(a, item, &r0, &r1);
    const int64_t q0 = a.tile_off[lo];
    if (j >= (int)(a.tile_off[lo + 1] - q0)) return;
    const int k = a.k, nv = a.ds >> 2;
    unsigned long long* out = a.partials + (size_t)unit * k;
    TopK tk{kEmpty, kEmpty};
    unsigned long long thr = topk_thr(tk, k);
    const float U = __uint_as_float(a.ufin[unit]);
    const float4* qrow = reinterpret_cast<const float4*>(a.Q + (size_t)a.qorder[q0 + j] * a.ds);
    float4 qv[NV];
#pragma unroll
    for (int u = 0; u < NV; ++u) {
        const int v = lane + 32 * u;
        qv[u] = v < nv ? __ldg(qrow + v) : make_float4(0.f, 0.f, 0.f, 0.f);
    }
    int rescored = 0;
    // rows of the set bits of nm: lane i of the warp holds row position rpos (from its entry);
    // kRB rows per round, their 16-byte loads in flight together (8 rows: 80 registers and a
    // stack frame, fewer warps, 0.95 -> 1.28 ms at c4, r02am; 4 kept)
    constexpr int kRB = 4;
    auto score_rows = [&](unsigned nm, uint32_t rpos) {
            while (nm) {
                uint32_t row[kRB];
                int nr = 0;
#pragma unroll
                for (int r = 0; r < kRB; ++r) {
                    row[r] = 0u;
                    if (nm) {
                        const int src = __ffs(nm) - 1;
                        nm &= nm - 1;
                        row[r] = (uint32_t)__shfl_sync(BLSH_FULL, rpos, src);
                        nr = r + 1;
                    }
                }
                float part[kRB];
#pragma unroll
                for (int r = 0; r < kRB; ++r) {
                    part[r] = 0.0f;
                    if (r < nr) {
                        const float4* xr = reinterpret_cast<const float4*>(a.Xp + (size_t)row[r] * a.ds);
#pragma unroll
                        for (int u = 0; u < NV; ++u) {
                            const int v = lane + 32 * u;
                            if (v < nv) {
                                const float4 x = __ldg(xr + v);
                                const float dx = qv[u].x - x.x, dy = qv[u].y - x.y, dz = qv[u].z - x.z, dw = qv[u].w - x.w;
                                part[r] = fmaf(dx, dx, part[r]);
                                part[r] = fmaf(dy, dy, part[r]);
                                part[r] = fmaf(dz, dz, part[r]);
                                part[r] = fmaf(dw, dw, part[r]);
                            }
                        }
                    }
                }
#pragma unroll
                for (int o = 16; o > 0; o >>= 1) {
#pragma unroll
                    for (int r = 0; r < kRB; ++r) part[r] += __shfl_xor_sync(BLSH_FULL, part[r], o);
                }
                uint32_t rl = row[0];
#pragma unroll
                for (int r = 1; r < kRB; ++r) rl = (lane & (kRB - 1)) == r ? row[r] : rl;
                const uint32_t idl = lane < nr ? __ldg(a.perm + rl) : 0u;
#pragma unroll
                for (int r = 0; r < kRB; ++r) {
                    const uint32_t id = __shfl_sync(BLSH_FULL, idl, r);
                    if (r < nr) {
                        const unsigned long long key = pack_entry(part[r], id);
                        if (key < thr) {
                            topk_insert(tk, key, lane);
                            thr = topk_thr(tk, k);
                        }
                    }
                }
            }
    };
    bool failed = false;
    for (int w = 0; w < a.nlist; ++w) failed |= a.scnt[unit * a.nlist + w] < 0;
    if (failed) {
        // The screen could not separate this query's candidates (a buffer overflowed):
        // exact distance to every row of the item whose query mask has bit j.
        const uint4* RI = a.rowinfo + a.rows_off[lo];
        for (int64_t base = r0; base < r1; base += 32) {
            const int64_t i = base + lane;
            const uint4 e = i < r1 ? RI[i] : make_uint4(0u, 0u, 0u, 0u);
            const unsigned nm = __ballot_sync(BLSH_FULL, (e.y >> j) & 1u);
            rescored += __popc(nm);
            score_rows(nm, e.x);
        }
    } else {
        // the buffered pairs list by list, 32 at a time, in the same order as a nested loop over
        // (list, batch); the next batch's entries are loaded while this batch is scored (the
        // entry load was the second largest stall line, 18% of samples, r02bb)
        const int nl = a.nlist;   // <= 8
        int cn[8];
#pragma unroll
        for (int w = 0; w < 8; ++w) cn[w] = w < nl ? a.scnt[unit * nl + w] : 0;
        auto cnt_of = [&](int w) {
            int c = cn[0];
#pragma unroll
            for (int x = 1; x < 8; ++x) c = w == x ? cn[x] : c;
            return c;
        };
        auto advance = [&](int& w, int& base) {   // the next non-empty batch after (w, base)
            base += 32;
            while (w < nl && base >= cnt_of(w)) { ++w; base = 0; }
        };
        auto load = [&](int w, int base) -> unsigned long long {
            if (w >= nl) return ~0ull;
            const int i = base + lane;
            return i < cnt_of(w) ? a.sbuf[((size_t)unit * nl + w) * a.scapw + i] : ~0ull;
        };
        int w = 0, base = -32;
        advance(w, base);
        unsigned long long e = load(w, base);
        while (w < nl) {
            int w2 = w, b2 = base;
            advance(w2, b2);
            const unsigned long long en = load(w2, b2);   // in flight while this batch is scored
            const int cnt = cnt_of(w);
            const int i = base + lane;
            // the k-th exact distance found so far bounds the final one too: once the list is
            // full, pairs whose lower bound exceeds it are skipped (ties: <= keeps them)
            const float dk = thr == kEmpty ? U : fminf(U, __uint_as_float((uint32_t)(thr >> 32)));
            const bool need = i < cnt && __uint_as_float((uint32_t)(e >> 32)) <= dk;
            const unsigned nm = __ballot_sync(BLSH_FULL, need);
            rescored += __popc(nm);
            score_rows(nm, (uint32_t)(e & 0xFFFFFFFFull));
            w = w2;
            base = b2;
            e = en;
        }
    }
    if (lane < k) out[lane] = tk.e0;
    if (lane + 32 < k) out[lane + 32] = tk.e1;
    if (lane == 0 && a.counters && rescored) atomicAdd(a.counters + 1, (unsigned long long)rescored);
}
