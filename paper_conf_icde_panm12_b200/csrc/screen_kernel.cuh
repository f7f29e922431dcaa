// screen_kernel.cuh -- the short-list screen on the compact fp16 table (a5), included
// by shortlist_tiled.cu inside its anonymous namespace after tc_kernel.cuh.
//
// Work item = (query tile of <= QT = 32 queries, range of the tile's candidate union).
// For a 128-row block of the union, one tcgen05.mma chain (kind::f16, M = 128,
// N = 48, K = dr in steps of 16, fp32 accumulators in TMEM) computes, per row i,
//   D_ij = r_i . u_j   (j < 32)    u_j = fp16((q_j - c) / S): the tile's centred queries
//   D_ia = r_i . v_a   (a < 16)    v_a = fp16((c - a) / S_v): the item's anchors seen from c
// straight from the fp16 residual rows r_i in shared memory (no conversion pass: the
// rows are copied by cp.async into the 128-byte-swizzled K-major layout the tensor core
// reads).  Every operand is a small difference vector (queries and anchors near c, rows
// near their anchor), so the tensor core's fp32 accumulation error stays far below the
// distances.  With x~ = a + s r (resid.cu) and K_aj = |q_j - a|^2 (k_anchor_k):
//   |q_j - x~|^2 = K_aj - 2 (q_j - c).(s r) - 2 (c - a).(s r) + |s r|^2
//               ~ K_aj + beta_i + m_i D_ij,
//   beta_i = nu_i - 2 S_v s D_i,a(i),   m_i = -2 S s.
// An item spans <= 16 anchor groups (k_tile_items), so every row's anchor has a column.
// Every rounding in that chain is bounded (DESIGN.md §7 "Screen bound"):
//   |d2(q_j, x_i) - d~2| <= delta d~2 + E_i + eta_j n_i,
// so lo = d~2 (1 - delta) - (E_i + eta_j n_i) <= d2 <= d~2 (1 + delta) + (E_i + eta_j n_i) = up.
// From there the epilogue is the one of k_shortlist_tc: lane j keeps query j's k smallest
// upper bounds (U_j), buffers every pair with lo <= U_j, and k_tc_rescore computes the
// exact fp32 distance of the survivors from the fp32 rows.  The screen only decides
// which pairs get exact work; results equal the warp short-list's.
//
// Warp roles (12 warps): 0 producer (bulk copies of swizzled 8-row atoms), 1 MMA issuer + TMEM
// allocation, 2-3 setup only, 4-11 epilogue (TMEM lane quadrant = warp % 4, two warps per
// quadrant, 16 rows each).

constexpr int kSxMma = 1;                   // MMA warp index
constexpr int kSxEpi0 = 4;                  // first epilogue warp
constexpr int kSxEpiN = 8;                  // epilogue warps: 2 per TMEM lane quadrant (16 rows each)
constexpr int kSxThreads = (kSxEpi0 + kSxEpiN) * 32;
constexpr int kSxAnc = 16;                  // anchor columns per item (items split at 16 anchor groups)
constexpr int kSxN = 32 + kSxAnc;           // MMA N: 32 queries + the item's anchors
constexpr uint32_t kSxStage = 128 * 128;    // one A stage: 128 rows x 64 fp16 columns (16 KB)
constexpr uint32_t kSxPanelB = kSxN * 128;  // one B panel: 48 rows x 64 fp16 columns (6 KB)
constexpr int kSxMaxK = 64;                 // k supported (per-lane bound lists of KT <= 64; the rescoring's warp top-k holds 64)
constexpr int kSxMaxDr = 512;            // (the setup stages the tile's queries in the A ring)
// A ring: NST stages of 16 KB (template: 8, or 6 / 4 when the B operand is large)
// instruction descriptor: D f32, A/B f16, K-major both, N = 48, M = 128
constexpr uint32_t kSxIdesc = (1u << 4) | ((uint32_t)(kSxN >> 3) << 17) | ((128u >> 4) << 24);
// error model (DESIGN.md §7 "Screen bound")
constexpr float kSxEpsAcc = 0x1p-14f;       // tensor-core fp32 accumulation, relative to sum |a_k b_k|
constexpr float kSxDelta = 0x1p-11f;        // relative slack on d~2 (AM-GM split 2^-12, K table 2^-13, fp32 ops)

// metadata ring depth: 8 (screen 5.09 -> 4.93 ms at c4: the producers' waits for the epilogue
// to release ring slots fell from 22 to 10 us per item; 6 / 7 slots or fetching 5-6 blocks
// ahead measured no better, r02ar); 8 fills the 227 KB of shared memory at d_r = 384, NST = 8
#ifndef BLSH_SX_NM   // (experiments: variant builds with -DBLSH_SX_NM=.. -DBLSH_SX_MA=..)
#define BLSH_SX_NM 8
#endif
#ifndef BLSH_SX_MA
#define BLSH_SX_MA 4
#endif
constexpr int kSxNM = BLSH_SX_NM;           // block metadata ring (row entries + bound constants)
constexpr int kSxMA = BLSH_SX_MA;           // metadata fetched this many blocks ahead of the producers

struct SxSmem {
    uint64_t afull[8], aempty[8];
    uint64_t tfull[4], tempty[4];
    uint64_t mfull[kSxNM], cfull[kSxNM], mempty[kSxNM];
    alignas(16) uint4 mrow[kSxNM][128];    // per block: (table row, query mask, K slot, -) of its 128 rows
    alignas(16) float4 mcon[kSxNM][128];   // per block: the rows' bound constants (resid.cu)
    uint32_t tmem_base;
    float S, Sv;
    float red[16], red2[16];
    float ca[kSxAnc];               // per anchor column: error constant of the D_ia term
    float kt[kSxAnc][QT];           // the item's K table rows: K_aj = |q_j - a|^2 (k_anchor_k)
    alignas(16) float eta[QT];
    uint32_t umin[QT];
    float ksub[kSxEpiN][QT];        // per epilogue warp and query: the ceil(k/8)-th smallest upper bound it has seen
    int scnt[kSxEpiN][QT];
    float tr[kSxEpiN][32 * 17];     // per epilogue warp: transposed dots [query][row of its 16]
    float4 rf[kSxEpiN][16];         // per epilogue warp and row: beta, m, E, n
    uint4 ru[kSxEpiN][16];          // per epilogue warp and row: mask, table row, K slot
    float cen[kSxMaxDr];            // tile centre c
};

__device__ __forceinline__ uint64_t sw128_desc(uint32_t saddr) {
    uint64_t d = 0;
    d |= (uint64_t)((saddr >> 4) & 0x3FFFu);
    d |= (uint64_t)1u << 16;                  // LBO (unused for swizzled K-major)
    d |= (uint64_t)(1024u >> 4) << 32;        // SBO: 8-row groups 1024 B apart
    d |= 1ull << 46;                          // descriptor version (sm_100)
    d |= 2ull << 61;                          // SWIZZLE_128B
    return d;
}
__device__ __forceinline__ void sx_mma(uint32_t d_tmem, uint64_t adesc, uint64_t bdesc, uint32_t accum) {
    asm volatile(
        "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
        "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(d_tmem),
        "l"(adesc), "l"(bdesc), "r"(kSxIdesc), "r"(accum)
        : "memory");
}
__device__ __forceinline__ void tmem_ld1(uint32_t taddr, float& a) {
    uint32_t r0;
    asm volatile("tcgen05.ld.sync.aligned.32x32b.x1.b32 {%0}, [%1];" : "=r"(r0) : "r"(taddr));
    asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
    a = __uint_as_float(r0);
}
// byte offset of 16-byte chunk ch of row n in a 128B-swizzled K-major panel
__device__ __forceinline__ uint32_t sw128_off(int n, int ch) {
    return (uint32_t)((n >> 3) * 1024 + (n & 7) * 128 + ((ch ^ (n & 7)) << 4));
}

// BLSH_TC_MODE & 32 (experiments): globaltimer stamps per item (0 start, 1 setup done, 2 producers done,
// 3 MMA done, 4 epilogue done, 5 end) and clock cycles spent waiting on mbarriers (6 producers on
// aempty, 7 MMA on afull, 8 MMA on tempty, 9 epilogue on tfull)
__device__ __forceinline__ void sx_stamp(const TiledArgs& a, int64_t item, int p) {
    if (a.tstamp) {
        unsigned long long t;
        asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
        a.tstamp[item * 16 + p] = t;
    }
}
// single-thread wait (no warp reconvergence: the caller is one lane)
__device__ __forceinline__ void mbar_wait1(uint64_t* bar, uint32_t parity) {
    asm volatile(
        "{\n\t.reg .pred p;\n"
        "WAIT1_%=:\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t"
        "@!p bra WAIT1_%=;\n\t}" ::"r"(smem_u32(bar)),
        "r"(parity)
        : "memory");
}
__device__ __forceinline__ void mbar_complete_tx(uint64_t* bar, uint32_t bytes) {
    asm volatile("mbarrier.complete_tx.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void sx_wait(const TiledArgs& a, uint64_t* bar, uint32_t parity, long long& acc) {
    if (a.tstamp) {
        const long long t0 = clock64();
        mbar_wait(bar, parity);
        acc += clock64() - t0;
    } else {
        mbar_wait(bar, parity);
    }
}

size_t screen_smem_bytes(int dr, int nst) {
    return 1024 + ((sizeof(SxSmem) + 1023) & ~size_t(1023)) + (size_t)(dr / 64) * kSxPanelB + (size_t)nst * kSxStage;
}
// the deepest A ring that fits (0: none)
int screen_stages(int dr) {
    for (int nst : {8, 6, 4})
        if (screen_smem_bytes(dr, nst) <= 227 * 1024) return nst;
    return 0;
}

template <int KT, int NST>
__global__ void __launch_bounds__(kSxThreads, 1) k_screen_f16(TiledArgs a) {
    constexpr int kSxNst = NST;
    extern __shared__ __align__(1024) unsigned char smraw_[];
    // the 128-byte-swizzled operands need 1024-byte aligned shared memory: align the base
    // (the launch reserves 1 KB for it) instead of trusting the declaration's alignment
    unsigned char* smraw = smraw_ + ((1024u - (smem_u32(smraw_) & 1023u)) & 1023u);
    SxSmem& S = *reinterpret_cast<SxSmem*>(smraw);
    const int ds = a.ds, dr = a.dr, np = dr >> 6;
    constexpr int nst = kSxNst;
    unsigned char* Bop = smraw + ((sizeof(SxSmem) + 1023) & ~size_t(1023));
    unsigned char* Aop = Bop + (size_t)np * kSxPanelB;
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const int64_t item = blockIdx.x;
    int64_t r0, r1;
    const int64_t tile = item_tile_rows(a, item, &r0, &r1);
    const int nblk = (int)((r1 - r0 + 127) / 128);
    const int k = a.k;
    const int64_t q0 = a.tile_off[tile];
    const int nqt = (int)(a.tile_off[tile + 1] - q0);
    const uint4* RI = a.rowinfo + a.rows_off[tile];
    if (threadIdx.x == 0) sx_stamp(a, item, 0);
    long long wcyc = 0;
    // ---- setup: centre c, scales, B operand (u_j, v_a), per-query eta ----
    // The tile's queries (rows 0..nqt-1) and the item's anchors (rows 32..) staged in shared
    // memory with a row pitch of dr floats (coalesced 16-byte loads; aliases the A ring, which
    // the producer only fills after the setup's last barrier).  Anchors beyond the ring's room
    // are read from global memory.
    float* Qf = reinterpret_cast<float*>(Aop);
    // the item's anchor slots: RI[r].z is non-decreasing; slot0 = its first, na <= kSxAnc
    const uint32_t slot0 = r1 > r0 ? RI[r0].z : 0u;
    const int na = r1 > r0 ? (int)(RI[r1 - 1].z - slot0) + 1 : 0;
    const int na_st = min(na, (int)((size_t)NST * kSxStage / ((size_t)dr * 4)) - 32);
    auto arow = [&](int la) -> const float* {
        return la < na_st ? Qf + (size_t)(32 + la) * dr : a.anc + (size_t)a.slot_anchor[slot0 + la] * dr;
    };
    {
        const int nv = ds >> 2, nvr = dr >> 2;
        for (int i = threadIdx.x; i < nqt * nv; i += kSxThreads) {
            const int n = i / nv, v = i - n * nv;
            reinterpret_cast<float4*>(Qf)[(size_t)n * nvr + v] =
                __ldg(reinterpret_cast<const float4*>(a.Q + (size_t)a.qorder[q0 + n] * ds) + v);
        }
        for (int i = threadIdx.x; i < na_st * nvr; i += kSxThreads) {
            const int la = i / nvr, v = i - la * nvr;
            reinterpret_cast<float4*>(Qf)[(size_t)(32 + la) * nvr + v] =
                __ldg(reinterpret_cast<const float4*>(a.anc + (size_t)a.slot_anchor[slot0 + la] * dr) + v);
        }
    }
    __syncthreads();
    for (int j = threadIdx.x; j < dr; j += kSxThreads) {
        float s = 0.f;
        if (j < ds)
            for (int n = 0; n < nqt; ++n) s += Qf[(size_t)n * dr + j];
        S.cen[j] = j < ds ? s / (float)nqt : 0.f;
    }
    __syncthreads();
    {   // S: max |q_jk - c_k|, S_v: max |c_k - a_k| over the item's anchors
        float mq = 0.f, mv = 0.f;
        for (int j = threadIdx.x; j < ds; j += kSxThreads) {
            const float c = S.cen[j];
            for (int n = 0; n < nqt; ++n) mq = fmaxf(mq, fabsf(Qf[(size_t)n * dr + j] - c));
            for (int la = 0; la < na; ++la) mv = fmaxf(mv, fabsf(c - arow(la)[j]));
        }
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) {
            mq = fmaxf(mq, __shfl_xor_sync(BLSH_FULL, mq, o));
            mv = fmaxf(mv, __shfl_xor_sync(BLSH_FULL, mv, o));
        }
        if (lane == 0) { S.red[warp] = mq; S.red2[warp] = mv; }
        __syncthreads();
        if (threadIdx.x < 2) {
            float m = 0.f;
            for (int w = 0; w < kSxThreads / 32; ++w) m = fmaxf(m, threadIdx.x ? S.red2[w] : S.red[w]);
            int e = 0;
            if (m > 0.f) { frexpf(m, &e); e -= 15; }
            const float sc = ldexpf(1.0f, max(-120, min(120, e)));
            if (threadIdx.x == 0) S.S = sc;
            else S.Sv = sc;
        }
        __syncthreads();
    }
    const float Sq = S.S, Sv = S.Sv;
    const float iSq = 1.0f / Sq, iSv = 1.0f / Sv;   // powers of two: exact
    for (int i = threadIdx.x; i < kSxN * (dr >> 3); i += kSxThreads) {
        const int n = i % kSxN, cc = i / kSxN;      // row n of B, 16-byte chunk cc (8 columns)
        __align__(16) __half h[8];
        const float* src = nullptr;
        if (n < nqt) src = Qf + (size_t)n * dr;
        else if (n >= 32 && n - 32 < na) src = arow(n - 32);
        float vv[8];
        if (src) {
            const float4 x0 = reinterpret_cast<const float4*>(src)[2 * cc];
            const float4 x1 = reinterpret_cast<const float4*>(src)[2 * cc + 1];
            vv[0] = x0.x; vv[1] = x0.y; vv[2] = x0.z; vv[3] = x0.w; vv[4] = x1.x; vv[5] = x1.y; vv[6] = x1.z; vv[7] = x1.w;
        }
#pragma unroll
        for (int e = 0; e < 8; ++e) {
            const int j = cc * 8 + e;
            float v = 0.f;
            if (j < ds && src) {
                const float c = S.cen[j];
                v = n < 32 ? (vv[e] - c) * iSq : (c - vv[e]) * iSv;
            }
            h[e] = __float2half_rn(v);
        }
        *reinterpret_cast<uint4*>(Bop + (size_t)(cc >> 3) * kSxPanelB + sw128_off(n, cc & 7)) =
            *reinterpret_cast<const uint4*>(h);
    }
    // per anchor column: |c - a| -> ca = error constant of 2 S_v s D_ia (accumulation, fp16
    // rounding of (c - a) / S_v, fp32 rounding of c - a, fp16 underflow)
    for (int la = warp; la < kSxAnc; la += kSxThreads / 32) {
        float sv = 0.f;
        if (la < na) {
            const float* ar = arow(la);
            for (int j = lane; j < ds; j += 32) {
                const float e = S.cen[j] - ar[j];
                sv = fmaf(e, e, sv);
            }
        }
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) sv += __shfl_xor_sync(BLSH_FULL, sv, o);
        if (lane == 0) {
            const float cn = sqrtf(sv) * (1.0f + 0x1p-18f);
            S.ca[la] = ((kSxEpsAcc + 0x1p-11f + 0x1p-23f) * (1.0f + 0x1p-9f) * cn + sqrtf((float)ds) * 0x1p-25f * Sv) *
                       (1.0f + 0x1p-10f);
        }
    }
    for (int i = threadIdx.x; i < na * QT; i += kSxThreads) S.kt[i / QT][i % QT] = __ldg(a.ktab + (size_t)slot0 * QT + i);
    for (int n = warp; n < QT; n += kSxThreads / 32) {
        float sq = 0.f, su = 0.f;
        if (n < nqt) {
            const float* qq = Qf + (size_t)n * dr;
            for (int j = lane; j < ds; j += 32) {
                const float e = qq[j] - S.cen[j];
                sq = fmaf(e, e, sq);
                const float u = __half2float(__float2half_rn(e * iSq));
                su = fmaf(u, u, su);
            }
        }
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) {
            sq += __shfl_xor_sync(BLSH_FULL, sq, o);
            su += __shfl_xor_sync(BLSH_FULL, su, o);
        }
        if (lane == 0) {
            const float qn = sqrtf(sq) * (1.0f + 0x1p-18f);
            const float un = sqrtf(su) * Sq * (1.0f + 0x1p-18f);
            const float om = (0x1p-11f + 0x1p-23f) * qn + sqrtf((float)ds) * 0x1p-25f * Sq;
            S.eta[n] = (2.0f * kSxEpsAcc * un + 2.0f * om + 0x1p-19f * (qn + om)) * (1.0f + 0x1p-10f);
        }
    }
    if (threadIdx.x < QT) S.umin[threadIdx.x] = 0x7F800000u;
    for (int i = threadIdx.x; i < kSxEpiN * QT; i += kSxThreads) (&S.ksub[0][0])[i] = __int_as_float(0x7F800000);
    if (threadIdx.x == 0) {
        for (int s = 0; s < nst; ++s) {
            mbar_init(&S.afull[s], 1);
            mbar_init(&S.aempty[s], 1);
        }
        for (int s = 0; s < 4; ++s) {
            mbar_init(&S.tfull[s], 1);
            mbar_init(&S.tempty[s], kSxEpiN);
        }
        for (int s = 0; s < kSxNM; ++s) {
            mbar_init(&S.mfull[s], 1);
            mbar_init(&S.cfull[s], 1);
            mbar_init(&S.mempty[s], kSxEpiN);
        }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    if (warp == kSxMma) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"(smem_u32(&S.tmem_base)));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");   // B operand visible to the tensor core
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tbase = S.tmem_base;
    const int nstage = nblk * np;
    if (threadIdx.x == 0) sx_stamp(a, item, 1);
    const int nrow = (int)(r1 - r0);

    if (warp == 0) {
        // ======================= producer (bulk copies) =======================
        // The item's rows are whole 8-row atoms (k_expand_atoms) and the fp16 table stores each
        // 64-column panel's atoms as consecutive swizzled KBs (resid.cu), so a 128-row stage is
        // one bulk copy per run of consecutive atoms among the block's 16 (lane i: run i; a
        // bucket is one run), completing by transaction bytes on afull.  Block metadata (the
        // block's 128 row entries, one contiguous 2 KB) is fetched kSxMA blocks ahead (mfull);
        // the rows' bound constants follow per run with the block's first stage (cfull).  No
        // thread waits on a dependent global load and nothing goes through the generic proxy.
        long long wa = 0, wme = 0, wmf = 0;
        const char* Rb = reinterpret_cast<const char*>(a.Rh);
        const size_t pstride = (size_t)a.natom * 1024;          // bytes per panel of the table
        auto fetch_meta = [&](int b) {                          // lane 0: block b's entries -> mrow
            if (b >= nblk) return;
            const int mb = b % kSxNM;
            if (b >= kSxNM) {
                const long long t0 = a.tstamp ? clock64() : 0;
                mbar_wait1(&S.mempty[mb], (uint32_t)(((b / kSxNM) - 1) & 1));
                if (a.tstamp) wme += clock64() - t0;
            }
            const int nr = min(128, nrow - b * 128);
            mbar_expect_tx(&S.mfull[mb], (uint32_t)nr * 16u);
            bulk_g2s(&S.mrow[mb][0], RI + r0 + (int64_t)b * 128, (uint32_t)nr * 16u, &S.mfull[mb]);
        };
        if (lane == 0)
            for (int b = 0; b < kSxMA; ++b) fetch_meta(b);
        __syncwarp();
        uint32_t ra = 0;                                        // the run this lane starts: first atom, length
        int rlen = 0, nat = 0;
        int b = 0, p = 0, slot = 0, sph = 0;                    // block, panel, ring slot, slot phase
        for (int g = 0; g < nstage; ++g) {
            const int mb = b % kSxNM;
            if (p == 0) {
                if (lane == 0) fetch_meta(b + kSxMA);
                sx_wait(a, &S.mfull[mb], (uint32_t)((b / kSxNM) & 1), wmf);
                nat = min(128, nrow - b * 128) >> 3;
                // runs of consecutive atoms: lane i < nat holds atom i (block rows 8i..8i+7); a run
                // starts where the atom does not follow its predecessor, and its first lane copies it
                const uint32_t at = lane < nat ? (S.mrow[mb][8 * lane].x >> 3) : 0u;
                const uint32_t prev = __shfl_up_sync(BLSH_FULL, at, 1);
                const bool start = lane < nat && (lane == 0 || prev + 1u != at);
                const unsigned sm = __ballot_sync(BLSH_FULL, start);
                const unsigned after = sm & ~((2u << lane) - 1u);      // run starts after this lane
                ra = at;
                rlen = start ? (after ? __ffs(after) - 1 : nat) - lane : 0;
                if (lane == 0) mbar_expect_tx(&S.cfull[mb], (uint32_t)nat * 128u);
                __syncwarp();
                if (rlen) bulk_g2s(&S.mcon[mb][8 * lane], a.rconst + (size_t)ra * 8, (uint32_t)rlen * 128u, &S.cfull[mb]);
            }
            // one release per slot (releasing slots in pairs, one commit per two stages, measured
            // slower: producer waits 17 us per item, screen 5.08 -> 5.44 ms at c4, r02an)
            if (g >= nst) sx_wait(a, &S.aempty[slot], (uint32_t)(sph ^ 1), wa);
            if (lane == 0) mbar_expect_tx(&S.afull[slot], (uint32_t)nat * 1024u);
            __syncwarp();
            if (rlen) {
                if (!(a.dbgmode & 2))
                    bulk_g2s(Aop + (size_t)slot * kSxStage + lane * 1024, Rb + p * pstride + (size_t)ra * 1024,
                             (uint32_t)rlen * 1024u, &S.afull[slot]);
                else
                    mbar_complete_tx(&S.afull[slot], (uint32_t)rlen * 1024u);   // ablation: no row loads
            }
            if (++p == np) { p = 0; ++b; }
            if (++slot == nst) { slot = 0; sph ^= 1; }
        }
        if (lane == 0 && a.tstamp) {
            sx_stamp(a, item, 2);
            a.tstamp[item * 16 + 6] = wa;
            a.tstamp[item * 16 + 10] = wmf;
            a.tstamp[item * 16 + 11] = wme;
        }
    } else if (warp == kSxMma) {
        // ======================= MMA issuer =======================
        long long wt = 0, wis = 0;
        for (int b = 0; b < nblk; ++b) {
            const int ts = b & 3;
            if (b >= 4) sx_wait(a, &S.tempty[ts], (uint32_t)(((b >> 2) - 1) & 1), wt);
            tc_fence_after();
            const uint32_t dt = tbase + (uint32_t)ts * 128u;
            for (int p = 0; p < np; ++p) {
                const int g = b * np + p;
                const int slot = g % nst;
                sx_wait(a, &S.afull[slot], (uint32_t)((g / nst) & 1), wcyc);
                tc_fence_after();
                if (lane == 0) {
                    const long long ti0 = a.tstamp ? clock64() : 0;
                    const uint32_t as = smem_u32(Aop + (size_t)slot * kSxStage);
                    const uint32_t bs = smem_u32(Bop + (size_t)p * kSxPanelB);
#pragma unroll
                    for (int kk = 0; kk < 4; ++kk)
                        if (!(a.dbgmode & 4))
                            sx_mma(dt, sw128_desc(as + 32u * kk), sw128_desc(bs + 32u * kk), (p > 0 || kk > 0) ? 1u : 0u);
                    tc_commit(&S.aempty[slot]);
                    if (p == np - 1) tc_commit(&S.tfull[ts]);
                    if (a.tstamp) wis += clock64() - ti0;
                }
                __syncwarp();
            }
        }
        if (lane == 0 && a.tstamp) {
            sx_stamp(a, item, 3);
            a.tstamp[item * 16 + 7] = wcyc;
            a.tstamp[item * 16 + 8] = wt;
            a.tstamp[item * 16 + 13] = wis;
        }
    } else if (warp >= kSxEpi0) {
        // ======================= epilogue =======================
        const int ew = warp - kSxEpi0;          // 0..7
        const int quad = warp & 3;              // TMEM lane quadrant of this warp
        const int half = ew >> 2;               // rows 16 half .. 16 half + 15 of the quadrant
        const bool mine_row = (lane >> 4) == half;
        const int j = lane;                     // query of this lane (screen phase)
        const float eta = S.eta[j];
        // Two valid bounds on query j's k-th smallest distance among the item's rows: the k-th
        // smallest upper bound one warp has seen (ulr[KT - 1]; any warp's), and -- since the 8
        // warps see disjoint rows -- the largest over the warps of each one's kk-th smallest,
        // kk = ceil(k / 8): every warp holds >= kk bounds below it, >= k in all.  The second is
        // near the true k-th (each warp sees 1/8 of the rows); the first is what a warp alone knows.
        // For k > KT (large k, KT = 64) a warp keeps only its kk smallest and only the second
        // bound is used.
        // (Used from KT = 32 on: at k <= 16 it buys few rescorings and costs screen time.)
        constexpr bool kSub = KT >= 32;
        const int kk = (k + kSxEpiN - 1) / kSxEpiN;
        const bool own_valid = k <= KT;
        const int klist = own_valid ? k : kk;   // real entries of the list
        const int isub = KT - klist + kk - 1;   // position of the kk-th smallest in the sorted list
        volatile float* ksub_all = &S.ksub[0][0];
        float ulr[KT];
#pragma unroll
        for (int p = 0; p < KT; ++p) ulr[p] = p < KT - klist ? __int_as_float(0xFF800000) : __int_as_float(0x7F800000);
        int my_cnt = 0, n_ins = 0, n_cmp = 0;
        long long wec = 0;
        bool my_fail = false;
        const int scapw = a.scapw;              // buffered pairs per (item, query, epilogue warp)
        unsigned long long* SBj = a.sbuf + (((size_t)item * QT + j) * kSxEpiN + ew) * scapw;
        float* Tt = S.tr[ew];
        for (int b = 0; b < nblk; ++b) {
            const int mb = b % kSxNM;
            const int ts = b & 3;
            sx_wait(a, &S.tfull[ts], (uint32_t)((b >> 2) & 1), wcyc);
            tc_fence_after();
            // this lane's row (row phase): entry and bound constants from the metadata ring
            sx_wait(a, &S.mfull[mb], (uint32_t)((b / kSxNM) & 1), wec);
            sx_wait(a, &S.cfull[mb], (uint32_t)((b / kSxNM) & 1), wec);
            const int rrow = quad * 32 + lane;
            const uint4 ri = b * 128 + rrow < nrow ? S.mrow[mb][rrow] : make_uint4(0u, 0u, 0u, 0u);
            const float4 rc = S.mcon[mb][rrow];
            const float sbv = rc.y;             // the group's scale s_g
            __syncwarp();
            if (lane == 0) mbar_arrive(&S.mempty[mb]);
            float dot[32];
            const uint32_t ta = tbase + ((uint32_t)(quad * 32) << 16) + (uint32_t)ts * 128u;
            tmem_ld32(ta, dot);
            // this row's anchor column 32 + la: one tcgen05.ld per distinct anchor among the 32 rows
            const bool live = ri.y != 0u;
            const int myla = (int)(ri.z - slot0);
            float Da = 0.f;
            unsigned pend = __ballot_sync(BLSH_FULL, live);
            while (pend) {
                const int la = __shfl_sync(BLSH_FULL, myla, __ffs(pend) - 1);
                float v;
                tmem_ld1(ta + 32u + (uint32_t)la, v);
                const bool mine = live && myla == la;
                if (mine) Da = v;
                pend &= ~__ballot_sync(BLSH_FULL, mine);
            }
            tc_fence_before();
            __syncwarp();
            if (lane == 0) mbar_arrive(&S.tempty[ts]);
            // per-row terms (lane = row)
            const float t2 = 2.0f * Sv * sbv * Da;
            const float beta = rc.x - t2;
            const float m = -2.0f * Sq * sbv;
            const float E = (2.0f * rc.z * (live ? S.ca[myla] : 0.f) + rc.w + 0x1p-21f * (fabsf(beta) + fabsf(t2))) *
                            (1.0f + 0x1p-10f);
            if (a.dbg && item == 0 && b == 0) {
                const int row = quad * 32 + lane;
                for (int jj = 0; jj < 32; ++jj) a.dbg[row * 32 + jj] = dot[jj];
                a.dbg[4096 + row] = Da;
                a.dbg[4096 + 128 + row] = (float)myla;
                a.dbg[4096 + 256 + row] = beta;
                a.dbg[4096 + 384 + row] = m;
                a.dbg[4096 + 512 + row] = E;
                a.dbg[4096 + 640 + row] = __uint_as_float(ri.x);
                a.dbg[4096 + 768 + row] = __uint_as_float(ri.y);
                a.dbg[4096 + 896 + row] = __uint_as_float(ri.z);
                if (row < 32) a.dbg[4096 + 1024 + row] = S.eta[row];
                a.dbg[4096 + 1152 + row] = rc.z;
                a.dbg[4096 + 1280 + row] = sbv;
                if (row == 0) {
                    a.dbg[4096 + 1056] = Sq; a.dbg[4096 + 1057] = Sv; a.dbg[4096 + 1058] = (float)na;
                    a.dbg[4096 + 1059] = (float)nqt;
                }
            }
            // transpose this warp's 16 rows: row lane writes its 32 dots, column j -> Tt[j][row]
            if (mine_row) {
                const int r16 = lane & 15;
#pragma unroll
                for (int jj = 0; jj < 32; ++jj) Tt[jj * 17 + r16] = dot[jj];
                S.rf[ew][r16] = make_float4(beta, m, E, rc.z);
                S.ru[ew][r16] = make_uint4(ri.y, ri.x, live ? (uint32_t)myla : 0u, 0u);   // K row: the item's anchor column
            }
            __syncwarp();
            if (a.dbgmode & 1) continue;                           // ablation: no screen loop
            float U = own_valid ? fminf(ulr[KT - 1], __uint_as_float(S.umin[j])) : __uint_as_float(S.umin[j]);
            if (kSub) {
                float us = ksub_all[j];
#pragma unroll
                for (int w = 1; w < kSxEpiN; ++w) us = fmaxf(us, ksub_all[w * QT + j]);
                if (us < U) {
                    U = us;
                    atomicMin(&S.umin[j], __float_as_uint(us));
                }
            }
            // pass 1 (branch-free): rows of this query whose lower bound clears the bound at the
            // block start; pass 2 takes them in row order against the tightening bound, so the
            // pairs kept are exactly those of a row-by-row loop
            auto row_bounds = [&](int i, float& lo, float& up) {
                const uint4 ru = S.ru[ew][i];                      // broadcast
                const float4 rf = S.rf[ew][i];
                const float d2 = S.kt[ru.z][j] + fmaf(rf.y, Tt[j * 17 + i], rf.x);
                const float err = fmaf(eta, rf.w, rf.z);
                lo = fmaf(d2, 1.0f - kSxDelta, -err);
                up = fmaf(d2, 1.0f + kSxDelta, err);
                return ru;
            };
            uint32_t pm = 0;
#pragma unroll
            for (int i = 0; i < 16; ++i) {
                float lo, up;
                const uint4 ru = row_bounds(i, lo, up);
                pm |= ((((ru.x >> j) & 1u) != 0u) && lo <= U) ? (1u << i) : 0u;
            }
            if (my_fail) pm = 0;
            while (pm) {
                const int i = __ffs(pm) - 1;
                pm &= pm - 1;
                float lo, up;
                const uint4 ru = row_bounds(i, lo, up);
                if (lo > U) continue;                              // the bound tightened since pass 1
                if (up < U) {                                      // sorted insert; only bounds below U matter
#pragma unroll
                    for (int p = KT - 1; p > 0; --p) ulr[p] = fmaxf(ulr[p - 1], fminf(ulr[p], up));
                    ulr[0] = fminf(ulr[0], up);
                    if (kSub) {
                        float sub = ulr[0];
#pragma unroll
                        for (int p = 1; p < KT; ++p) sub = p == isub ? ulr[p] : sub;
                        ksub_all[ew * QT + j] = sub;               // only decreases: stale reads stay valid
                    }
                    if (own_valid && ulr[KT - 1] < U) {            // share the tighter bound at once
                        U = ulr[KT - 1];
                        atomicMin(&S.umin[j], __float_as_uint(U));
                    }
                }
                const unsigned long long e = ((unsigned long long)__float_as_uint(fmaxf(lo, 0.f)) << 32) | ru.y;
                ++n_ins;
                if (my_cnt == scapw) {                             // full: drop what the tighter U excludes
                    ++n_cmp;
                    int c2 = 0;
                    const ulonglong2* B2 = reinterpret_cast<const ulonglong2*>(SBj);
                    for (int t0 = 0; t0 < scapw / 2; t0 += 8) {    // 8 independent 16-byte loads per batch
                        ulonglong2 f[8];
#pragma unroll
                        for (int u = 0; u < 8; ++u) f[u] = B2[t0 + u];
#pragma unroll
                        for (int u = 0; u < 8; ++u) {
                            if (__uint_as_float((uint32_t)(f[u].x >> 32)) <= U) SBj[c2++] = f[u].x;
                            if (__uint_as_float((uint32_t)(f[u].y >> 32)) <= U) SBj[c2++] = f[u].y;
                        }
                    }
                    my_cnt = c2;
                    if (my_cnt > 3 * scapw / 4) { my_fail = true; break; }     // exact scan of j's rows later
                }
                SBj[my_cnt++] = e;
            }
            __syncwarp();                                          // Tt / rf / ru reused by the next block
        }
        S.scnt[ew][j] = my_fail ? -1 : my_cnt;
        if (warp == kSxEpi0 && lane == 0 && a.tstamp) {
            sx_stamp(a, item, 4);
            a.tstamp[item * 16 + 9] = wcyc;
            a.tstamp[item * 16 + 12] = wec;
        }
        if (a.counters && my_cnt) atomicAdd(a.counters, (unsigned long long)my_cnt);   // kept pairs
        if (a.counters && n_ins) atomicAdd(a.counters + 2, (unsigned long long)n_ins);   // buffer insertions
        if (a.counters && n_cmp) atomicAdd(a.counters + 3, (unsigned long long)n_cmp);   // compactions
        if (a.counters && my_fail) atomicAdd(a.counters + 4, 1ull);                       // overflowed lists
    }
    tc_fence_before();
    __syncthreads();
    if (warp == kSxMma) {
        tc_fence_after();
        asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" ::"r"(tbase));
    }
    if (threadIdx.x == 0) sx_stamp(a, item, 5);
    // ---- hand-off to k_tc_rescore: final bound U_j, buffered pair counts ----
    if (threadIdx.x < QT) {
        const int j = threadIdx.x;
        a.ufin[(size_t)item * QT + j] = j < nqt ? S.umin[j] : 0u;
#pragma unroll
        for (int w = 0; w < kSxEpiN; ++w)
            a.scnt[((size_t)item * QT + j) * kSxEpiN + w] = j < nqt ? min(S.scnt[w][j], a.scapw) : 0;
    }
}

// K_aj = |q_j - a|^2 for every (tile, anchor slot): one CTA per tile, the tile's queries
// staged in shared memory (row pitch ds + 4 floats: conflict-free float4 reads), one warp
// per anchor slot, lane j = query j, fp32 direct form in 4 partial chains.
__global__ void __launch_bounds__(256) k_anchor_k(const float* __restrict__ Q, int ds, const uint32_t* __restrict__ qorder,
                                                  const int64_t* __restrict__ tile_off, const int64_t* __restrict__ aoff,
                                                  const uint32_t* __restrict__ slot_anchor, const float* __restrict__ anc,
                                                  int dr, float* __restrict__ ktab) {
    extern __shared__ float4 qs4[];
    const int64_t t = blockIdx.x;
    const int64_t q0 = tile_off[t];
    const int nqt = (int)(tile_off[t + 1] - q0);
    const int nv = ds >> 2, pitch = nv + 1;
    for (int i = threadIdx.x; i < QT * nv; i += 256) {
        const int n = i / nv, v = i - n * nv;
        qs4[n * pitch + v] = n < nqt ? __ldg(reinterpret_cast<const float4*>(Q + (size_t)qorder[q0 + n] * ds) + v)
                                     : make_float4(0.f, 0.f, 0.f, 0.f);
    }
    __syncthreads();
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const float4* qr = qs4 + lane * pitch;
    for (int64_t sl = aoff[t] + warp; sl < aoff[t + 1]; sl += 8) {
        const float4* ar = reinterpret_cast<const float4*>(anc + (size_t)slot_anchor[sl] * dr);
        float s0 = 0.f, s1 = 0.f, s2 = 0.f, s3 = 0.f;
        for (int v = 0; v < nv; ++v) {
            const float4 x = __ldg(ar + v), q = qr[v];
            const float e0 = q.x - x.x, e1 = q.y - x.y, e2 = q.z - x.z, e3 = q.w - x.w;
            s0 = fmaf(e0, e0, s0);
            s1 = fmaf(e1, e1, s1);
            s2 = fmaf(e2, e2, s2);
            s3 = fmaf(e3, e3, s3);
        }
        ktab[(size_t)sl * QT + lane] = lane < nqt ? (s0 + s1) + (s2 + s3) : 0.f;
    }
}

// ---------------------------------------------------------------------------
// Large k (64 < k <= kSxMaxKLarge, the paper's k = 500 of P:217) after the fp16 screen:
// every surviving (row, query) pair of a work item gets its exact fp32 distance (the warp
// short-list's form, R22) and its packed (d^2, id) key goes to the query's key segment;
// launch_select then keeps the k smallest per query (as the warp large-k path does).
//   k_unit_counts    keys per (item, query) unit: its buffered pairs, or (a buffer
//                    overflowed) every row of the item whose query mask has bit j
//   k_query_counts   per query: total over its tile's items, each unit's offset in it
//   k_tc_emit        one warp per unit: exact distances, keys at the unit's offset;
//                    buffered pairs the final bound excludes become padding keys
// ---------------------------------------------------------------------------
constexpr int kSxMaxKLarge = 512;   // kk = ceil(k / 8) <= 64: the KT = 64 lists hold it

__global__ void __launch_bounds__(256) k_unit_counts(TiledArgs a, int64_t* __restrict__ ucnt) {
    const int lane = threadIdx.x & 31;
    const int64_t unit = blockIdx.x * (int64_t)8 + (threadIdx.x >> 5);
    if (unit >= a.n_items * QT) return;
    const int64_t item = unit / QT;
    const int j = (int)(unit % QT);
    int64_t r0, r1;
    const int64_t t = item_tile_rows(a, item, &r0, &r1);
    if (j >= (int)(a.tile_off[t + 1] - a.tile_off[t])) {
        if (lane == 0) ucnt[unit] = 0;
        return;
    }
    bool failed = false;
    int64_t c = 0;
    for (int w = 0; w < a.nlist; ++w) {
        const int v = a.scnt[unit * a.nlist + w];
        failed |= v < 0;
        c += v > 0 ? v : 0;
    }
    if (failed) {
        const uint4* RI = a.rowinfo + a.rows_off[t];
        c = 0;
        for (int64_t base = r0; base < r1; base += 32) {
            const int64_t i = base + lane;
            const uint4 e = i < r1 ? RI[i] : make_uint4(0u, 0u, 0u, 0u);
            c += __popc(__ballot_sync(BLSH_FULL, (e.y >> j) & 1u));
        }
    }
    if (lane == 0) ucnt[unit] = c;
}

__global__ void __launch_bounds__(256) k_query_counts(TiledArgs a, const int64_t* __restrict__ ucnt,
                                                      int64_t* __restrict__ uloc, int64_t* __restrict__ qcnt) {
    const int64_t pos = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (pos >= a.nq) return;
    const int64_t t = a.tile_of[pos];
    const int j = (int)(pos - a.tile_off[t]);
    int64_t c = 0;
    for (int64_t it = a.item_off[t]; it < a.item_off[t + 1]; ++it) {
        uloc[it * QT + j] = c;
        c += ucnt[it * QT + j];
    }
    qcnt[a.qorder[pos]] = c;
}

template <int NV>
__global__ void __launch_bounds__(256) k_tc_emit(TiledArgs a, const int64_t* __restrict__ uloc,
                                                 const int64_t* __restrict__ cand_off,
                                                 unsigned long long* __restrict__ keys) {
    const int lane = threadIdx.x & 31;
    const int64_t unit = blockIdx.x * (int64_t)8 + (threadIdx.x >> 5);
    if (unit >= a.n_items * QT) return;
    const int64_t item = unit / QT;
    const int j = (int)(unit % QT);
    int64_t r0, r1;
    const int64_t t = item_tile_rows(a, item, &r0, &r1);
    const int64_t q0 = a.tile_off[t];
    if (j >= (int)(a.tile_off[t + 1] - q0)) return;
    const int nv = a.ds >> 2;
    const uint32_t qid = a.qorder[q0 + j];
    unsigned long long* seg = keys + cand_off[qid] + uloc[unit];
    const float U = __uint_as_float(a.ufin[unit]);
    const float4* qrow = reinterpret_cast<const float4*>(a.Q + (size_t)qid * a.ds);
    float4 qv[NV];
#pragma unroll
    for (int u = 0; u < NV; ++u) {
        const int v = lane + 32 * u;
        qv[u] = v < nv ? __ldg(qrow + v) : make_float4(0.f, 0.f, 0.f, 0.f);
    }
    int rescored = 0;
    // rows of the set bits of nm (lane i holds row position rpos); row r of a group goes to
    // slot sbase + (compact ? its rank among the set bits : its source lane)
    auto score_rows = [&](unsigned nm, uint32_t rpos, int64_t sbase, bool compact) {
        int done = 0;
        while (nm) {
            uint32_t row[4];
            int src[4];
            int nr = 0;
#pragma unroll
            for (int r = 0; r < 4; ++r) {
                row[r] = 0u;
                src[r] = 0;
                if (nm) {
                    src[r] = __ffs(nm) - 1;
                    nm &= nm - 1;
                    row[r] = (uint32_t)__shfl_sync(BLSH_FULL, rpos, src[r]);
                    nr = r + 1;
                }
            }
            float part[4];
#pragma unroll
            for (int r = 0; r < 4; ++r) {
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
                for (int r = 0; r < 4; ++r) part[r] += __shfl_xor_sync(BLSH_FULL, part[r], o);
            }
            const uint32_t rl = (lane & 3) == 0 ? row[0] : (lane & 3) == 1 ? row[1] : (lane & 3) == 2 ? row[2] : row[3];
            const uint32_t idl = lane < nr ? __ldg(a.perm + rl) : 0u;
#pragma unroll
            for (int r = 0; r < 4; ++r) {
                const uint32_t id = __shfl_sync(BLSH_FULL, idl, r);
                if (r < nr && lane == r) seg[sbase + (compact ? done + r : src[r])] = pack_entry(part[r], id);
            }
            done += nr;
        }
    };
    bool failed = false;
    for (int w = 0; w < a.nlist; ++w) failed |= a.scnt[unit * a.nlist + w] < 0;
    if (failed) {
        const uint4* RI = a.rowinfo + a.rows_off[t];
        int64_t at = 0;
        for (int64_t base = r0; base < r1; base += 32) {
            const int64_t i = base + lane;
            const uint4 e = i < r1 ? RI[i] : make_uint4(0u, 0u, 0u, 0u);
            const unsigned nm = __ballot_sync(BLSH_FULL, (e.y >> j) & 1u);
            rescored += __popc(nm);
            score_rows(nm, e.x, at, true);
            at += __popc(nm);
        }
    } else {
        int64_t at = 0;
        for (int w = 0; w < a.nlist; ++w) {
            const int cnt = a.scnt[unit * a.nlist + w];
            const unsigned long long* Bf = a.sbuf + ((size_t)unit * a.nlist + w) * a.scapw;
            for (int base = 0; base < cnt; base += 32) {
                const int i = base + lane;
                const unsigned long long e = i < cnt ? Bf[i] : ~0ull;
                const bool need = i < cnt && __uint_as_float((uint32_t)(e >> 32)) <= U;
                if (i < cnt && !need) seg[at + lane] = kEmpty;     // excluded by the final bound: padding
                const unsigned nm = __ballot_sync(BLSH_FULL, need);
                rescored += __popc(nm);
                score_rows(nm, (uint32_t)(e & 0xFFFFFFFFull), at, false);
                at += min(32, cnt - base);
            }
        }
    }
    if (lane == 0 && a.counters && rescored) atomicAdd(a.counters + 1, (unsigned long long)rescored);
}
