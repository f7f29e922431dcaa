// probe_kernel.cuh -- a3 + a4, one warp per query (included by query.cu inside
// its anonymous namespace, after warp_select / find_bucket / lat_score).
//
// Z^M path templated on M so the perturbation pool lives in registers:
// per coordinate the admissible options among {-1, 0, +1} (those whose term
// x_i(delta)^2 is <= the bound B' of DESIGN.md §7), decoded from the pool
// index with divisions by 1, 2 or 3 (multiply-high), least-significant
// coordinate first; the score is then summed in ascending coordinate order
// (R11), exactly as the oracle does.

template <int MM>
struct PoolT {
    double sqm[MM], sqp[MM];   // x_i(-1)^2, x_i(+1)^2 (exact products of fp32 values)
    uint32_t nopt[MM];         // 1..3 options per coordinate
    uint32_t hasm[MM];         // 1 if -1 is an option
    uint32_t P, home;
};

template <int MM>
__device__ __forceinline__ double pool_score(const PoolT<MM>& pl, uint32_t x, int8_t* dl) {
    int8_t d[MM];
#pragma unroll
    for (int i = MM - 1; i >= 0; --i) {
        const uint32_t n = pl.nopt[i];
        const uint32_t qv = n == 3u ? (__umulhi(x, 0xAAAAAAABu) >> 1) : (n == 2u ? (x >> 1) : x);
        d[i] = (int8_t)((int)(x - qv * n) - (int)pl.hasm[i]);
        x = qv;
    }
    double s = 0.0;
#pragma unroll
    for (int i = 0; i < MM; ++i) {
        if (d[i] < 0) s = __dadd_rn(s, pl.sqm[i]);
        else if (d[i] > 0) s = __dadd_rn(s, pl.sqp[i]);
        dl[i] = d[i];
    }
    return s;
}

// Every perturbation delta != 0 with score(delta) <= Bp, in enc order, by a
// breadth-first expansion over the coordinates (i ascending): a partial
// assignment keeps its running sum, which is exactly the score's summation
// order (R11), and is dropped as soon as the sum exceeds Bp (rounded sums of
// non-negative terms never decrease, so no completion of it can come back under
// Bp).  Children are written in digit order after a warp scan, so each level is
// sorted by enc prefix.  Returns false when a level would exceed kFCap.
template <int MM>
__device__ bool frontier_enum(ProbeSmem& sm, const PoolT<MM>& pl, double Bp, int lane, int* K, int* buf) {
    int F = 1, cur = 0;
    uint32_t home = 0;                  // enc prefix of the all-zero partial
    if (lane == 0) {
        sm.fs[0][0] = 0.0;
        sm.fe[0][0] = 0u;
    }
    __syncwarp();
#pragma unroll
    for (int i = 0; i < MM; ++i) {
        const bool last = i == MM - 1;
        int out = 0;
        for (int base = 0; base < F; base += 32) {
            const int e = base + lane;
            const bool v = e < F;
            const double sp = v ? sm.fs[cur][e] : 0.0;
            const uint32_t en = v ? sm.fe[cur][e] : 0u;
            const double sm1 = __dadd_rn(sp, pl.sqm[i]), sp1 = __dadd_rn(sp, pl.sqp[i]);
            const bool cm = v && sm1 <= Bp;
            const bool c0 = v && !(last && en == home);
            const bool cp = v && sp1 <= Bp;
            const int c = (int)cm + (int)c0 + (int)cp;
            int inc = c;
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                const int y = __shfl_up_sync(BLSH_FULL, inc, o);
                if (lane >= o) inc += y;
            }
            const int tot = __shfl_sync(BLSH_FULL, inc, 31);
            if (out + tot > kFCap) return false;
            int at = out + inc - c;
            const int nx = cur ^ 1;
            if (cm) { sm.fs[nx][at] = sm1; sm.fe[nx][at] = en * 3u; ++at; }
            if (c0) { sm.fs[nx][at] = sp; sm.fe[nx][at] = en * 3u + 1u; ++at; }
            if (cp) { sm.fs[nx][at] = sp1; sm.fe[nx][at] = en * 3u + 2u; }
            out += tot;
        }
        home = home * 3u + 1u;
        F = out;
        cur ^= 1;
        __syncwarp();
    }
    *K = F;
    *buf = cur;
    return true;
}

template <int MM>
__device__ int64_t probe_zm(const QueryArgs& a, ProbeSmem& sm, int64_t q, int lane, int64_t ulo, int64_t uhi,
                            uint2* ivl) {
    const int T = a.T, B = a.B;
    const float* tq = a.qt + (size_t)q * MM;
    float t[MM], fl[MM];
#pragma unroll
    for (int i = 0; i < MM; ++i) {
        t[i] = tq[i];
        fl[i] = floorf(t[i]);
    }
    PoolT<MM> pl;
    int fbuf = -1;                // >= 0: the selection indexes the frontier sm.fe[fbuf]
    if (a.probe == 1 && T > 1) {
        double v[2 * MM];
#pragma unroll
        for (int i = 0; i < MM; ++i) {
            const float xm = __fsub_rn(t[i], fl[i]);
            const float xp = __fsub_rn(1.0f, xm);
            pl.sqm[i] = (double)xm * (double)xm;
            pl.sqp[i] = (double)xp * (double)xp;
            v[2 * i] = pl.sqm[i];
            v[2 * i + 1] = pl.sqp[i];
        }
        // bound B': sum of the J smallest terms, J minimal with >= T-1 valid subsets.
        // Lane j < 2M holds term j and its rank in the order (value, index); the
        // J-th smallest is then one ballot away (the same sequence a selection
        // by smallest value, lowest index first, takes).
        double vme = 0.0;
#pragma unroll
        for (int j = 0; j < 2 * MM; ++j)
            if (lane == j) vme = v[j];
        int rank = 0;
#pragma unroll
        for (int j = 0; j < 2 * MM; ++j) {
            const double vj = __shfl_sync(0xFFFFFFFFu, vme, j);
            rank += (vj < vme || (vj == vme && j < lane)) ? 1 : 0;
        }
        if (lane >= 2 * MM) rank = 64;
        uint32_t used = 0;            // 2 bits per coordinate
        double Bsum = 0.0;
        for (int J = 0; J < 2 * MM; ++J) {
            const int jb = __ffs(__ballot_sync(0xFFFFFFFFu, rank == J)) - 1;
            if (jb < 0) break;   // NaN terms (no rank J): stop at the terms ranked so far
            const double vb = __shfl_sync(0xFFFFFFFFu, vme, jb);
            used += 1u << (2 * (jb >> 1));
            Bsum = __dadd_rn(Bsum, vb);
            uint32_t prod = 1;
#pragma unroll
            for (int i = 0; i < MM; ++i) prod *= 1u + ((used >> (2 * i)) & 3u);
            if (prod - 1u >= (uint32_t)(T - 1)) break;
        }
        const double Bp = __dmul_ru(Bsum, 1.0 + 0x1p-40);
        uint32_t P = 1, home = 0;
#pragma unroll
        for (int i = MM - 1; i >= 0; --i) {
            const uint32_t hm = pl.sqm[i] <= Bp ? 1u : 0u;
            const uint32_t hp = pl.sqp[i] <= Bp ? 1u : 0u;
            pl.hasm[i] = hm;
            pl.nopt[i] = 1u + hm + hp;
            home += hm * P;
            P *= pl.nopt[i];
        }
        pl.P = P;
        pl.home = home;
        int K = 0;
        if (MM <= 10 && frontier_enum<MM>(sm, pl, Bp, lane, &K, &fbuf)) {
            warp_select(sm, (uint32_t)K, 0xFFFFFFFFu, T - 1, [&](uint32_t x) { return sm.fs[fbuf][x]; });
        } else {
            fbuf = -1;
            warp_select(sm, P, home, T - 1, [&](uint32_t x) {
                int8_t dl[MM];
                return pool_score<MM>(pl, x, dl);
            });
        }
    }
    int64_t mysum = 0;
    const float lo = -(float)(1 << (B - 1)), hi = (float)((1 << (B - 1)) - 1);
    for (int p = lane; p < T; p += 32) {
        int8_t dl[MM];
#pragma unroll
        for (int i = 0; i < MM; ++i) dl[i] = 0;
        bool sel_ok = true;
        if (p > 0 && sm.order[p - 1] == 0xFFFFFFFFu) sel_ok = false;   // short pool (warp_select)
        else if (p > 0) {
            if (fbuf >= 0) {
                uint32_t en = sm.fe[fbuf][sm.order[p - 1]];
#pragma unroll
                for (int i = MM - 1; i >= 0; --i) {
                    const uint32_t qv = __umulhi(en, 0xAAAAAAABu) >> 1;
                    dl[i] = (int8_t)((int)(en - qv * 3u) - 1);
                    en = qv;
                }
            } else {
                pool_score<MM>(pl, sm.order[p - 1], dl);
            }
        }
        int32_t pc[MM];
        bool valid = sel_ok;
#pragma unroll
        for (int i = 0; i < MM; ++i) {
            const float f = __fadd_rn(fl[i], (float)dl[i]);
            if (!(f >= lo && f <= hi)) valid = false;
            pc[i] = valid ? (int32_t)f : 0;
        }
        Key128 k{0, 0};
        uint2 iv = make_uint2(0, 0);
        if (valid) {
            k = morton_key(pc, MM, B);
            const int64_t u = find_bucket(a.ukey, ulo, uhi, k);
            if (u >= 0) iv = make_uint2(a.uoff[u], a.uoff[u + 1]);
        }
        ivl[p] = iv;
        mysum += (int64_t)(iv.y - iv.x);
        if (a.pkey) {
            a.pkey[(size_t)q * T + p] = k;
            a.pvalid[(size_t)q * T + p] = valid ? 1 : 0;
        }
    }
    return mysum;
}

__device__ int64_t probe_e8(const QueryArgs& a, ProbeSmem& sm, int64_t q, int lane, int oor, int64_t ulo,
                            int64_t uhi, uint2* ivl) {
    const int T = a.T, B = a.B, M = a.M;   // M = 8, or 16 = two E8 blocks (R28)
    const float* t = a.qt + (size_t)q * M;
    const int32_t* code = a.qcode + (size_t)q * M;
    if (M == 8 && a.probe == 2 && T > 241 && !(oor & 1)) {   // recursive probing (R26): the second ring
        warp_select(sm, 9120u, 0xFFFFFFFFu, T - 241, [&](uint32_t x) { return ring2_score(t, code, x); });
        if (lane < T - 241) sm.order2[lane] = sm.order[lane];
        __syncwarp();
    }
    if (a.probe == 2 && T > 1 && !(oor & 1)) {
        if (M == 8) warp_select(sm, 240u, 0xFFFFFFFFu, min(T - 1, 240), [&](uint32_t x) { return lat_score(t, code, x); });
        else warp_select(sm, 480u, 0xFFFFFFFFu, T - 1, [&](uint32_t x) { return lat2_score(t, code, x); });
    }
    int64_t mysum = 0;
    // R33 ("if the number of candidates computed is not enough, we recursively probe the
    // adjacent buckets of the 240 probed buckets"): with rec_tau > 0 the second-ring probes
    // p = 241..T-1 (T <= 256: the last lane-strided round, lane = p - 224) are looked up first and
    // decided after the loop: probe p is taken iff the probes before it hold < rec_tau candidates.
    const bool rec = a.rec_tau > 0 && M == 8 && T > 241;
    Key128 rk{0, 0};
    uint2 riv = make_uint2(0, 0);
    bool rvalid = false, rpend = false;
    for (int p = lane; p < T; p += 32) {
        int32_t pc[16];
        bool valid = !(oor & 1);
        for (int i = 0; i < M; ++i) pc[i] = code[i];
        if (p > 0 && valid) {
            if (M == 8) {
                const bool ring = p > 240;
                const uint32_t r = ring ? sm.order2[p - 241] : sm.order[p - 1];
                if (r == 0xFFFFFFFFu) valid = false;   // short pool (warp_select)
                else {
#pragma unroll
                    for (int i = 0; i < 8; ++i) pc[i] += ring ? (int32_t)g_e8_ring2[r][i] : (int32_t)c_e8_roots[r][i];
                }
            } else {
                const uint32_t x = sm.order[p - 1], blk = x / 240u, r = x - blk * 240u;
                if (x == 0xFFFFFFFFu) valid = false;
                else {
#pragma unroll
                    for (int i = 0; i < 8; ++i) pc[8 * blk + i] += (int32_t)c_e8_roots[r][i];
                }
            }
        }
        const int32_t lo = -(1 << (B - 1)), hi = (1 << (B - 1)) - 1;
        if (valid)
            for (int i = 0; i < M; ++i)
                if (pc[i] < lo || pc[i] > hi) valid = false;
        Key128 k{0, 0};
        uint2 iv = make_uint2(0, 0);
        if (valid) {
            k = morton_key(pc, M, B);
            const int64_t u = find_bucket(a.ukey, ulo, uhi, k);
            if (u >= 0) iv = make_uint2(a.uoff[u], a.uoff[u + 1]);
        }
        if (rec && p > 240) {   // decided below
            rk = k; riv = iv; rvalid = valid; rpend = true;
            continue;
        }
        ivl[p] = iv;
        mysum += (int64_t)(iv.y - iv.x);
        if (a.pkey) {
            a.pkey[(size_t)q * T + p] = k;
            a.pvalid[(size_t)q * T + p] = valid ? 1 : 0;
        }
    }
    if (rec) {
        int64_t before = mysum;                       // probes 0..240: every lane's sum
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) before += __shfl_xor_sync(BLSH_FULL, before, o);
        const int64_t sz = rpend ? (int64_t)(riv.y - riv.x) : 0;
        int64_t inc = sz;                             // inclusive scan over lanes = ring probes in order
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const int64_t v = __shfl_up_sync(BLSH_FULL, inc, o);
            if (lane >= o) inc += v;
        }
        if (rpend) {
            const int p = lane + 224;
            const bool take = before + (inc - sz) < a.rec_tau;
            const uint2 iv = take ? riv : make_uint2(0, 0);
            ivl[p] = iv;
            mysum += (int64_t)(iv.y - iv.x);
            if (a.pkey) {
                a.pkey[(size_t)q * T + p] = take && rvalid ? rk : Key128{0, 0};
                a.pvalid[(size_t)q * T + p] = take && rvalid ? 1 : 0;
            }
        }
    }
    return mysum;
}

// probe = 3, Morton-curve neighbours ("search within the Morton curve to
// find the position where the query code can be inserted without violating the
// ordering ... use the Morton codes before and after the insert position ...
// to refer the buckets").  Reading R25: p = the insertion position of the
// query's clamped home key among its leaf's sorted bucket keys (lower bound);
// probe j takes bucket p + o_j with o = 0, -1, +1, -2, +2, ... (after, before,
// alternating: T = 2 is exactly "before and after"; when the key is present,
// bucket p is its home bucket); offsets outside the leaf are empty probes that
// count toward T.  Every probe is one whole bucket, so the intervals are
// disjoint (and the hierarchy's containment rule applies unchanged).
//
// R31 ("perturb some bits of the query Morton code and repeat this process
// several times [23]"): with P = a.cperturb > 0 the search is repeated for the keys
// kappa_r = home key with bit 0 of coordinate c_r flipped (key bit M-1-c_r: one cell
// towards +1 when that bit is 0, else towards -1), c_1, c_2, .. = the coordinates by
// ascending (x_i(delta_i), i) (R11's boundary distances, fp32); probe j searches around
// key j mod (P+1) with offset number j div (P+1); a bucket already probed by an earlier
// probe is an empty probe (the intervals stay disjoint).
__device__ __forceinline__ int64_t curve_lower(const QueryArgs& a, int64_t lo, int64_t hi, const Key128& k) {
    while (lo < hi) {   // every lane that calls it runs the same search (keys L1/L2-resident)
        const int64_t mid = (lo + hi) >> 1;
        if (key_lt(a.ukey[mid], k)) lo = mid + 1;
        else hi = mid;
    }
    return lo;
}

__device__ int64_t probe_curve(const QueryArgs& a, int64_t q, int lane, int64_t ulo, int64_t uhi, uint2* ivl) {
    const int T = a.T, M = a.M;
    const int R = a.cperturb + 1;
    const Key128 k = a.qkey[q];
    const int64_t p0 = curve_lower(a, ulo, uhi, k);
    // perturbed keys: lane i < M owns coordinate i; its rank among the coordinates decides
    // which key (r = rank + 1) it holds, and it searches that key's insertion position
    int64_t pmine = p0;
    int rank = 32;
    if (R > 1) {
        float xd = 0.f;
        if (lane < M) {
            const float t = a.qt[(size_t)q * M + lane];
            const float xm = __fsub_rn(t, floorf(t));                      // x_i(-1)
            const bool up = ((k.lo >> (M - 1 - lane)) & 1ull) == 0ull;       // bit 0 of u_i
            xd = up ? __fsub_rn(1.0f, xm) : xm;
        }
        rank = 0;
        for (int j = 0; j < M; ++j) {
            const float xj = __shfl_sync(BLSH_FULL, xd, j);
            rank += (xj < xd || (xj == xd && j < lane)) ? 1 : 0;
        }
        if (lane < M && rank < R - 1) {
            const Key128 kp{k.hi, k.lo ^ (1ull << (M - 1 - lane))};
            pmine = curve_lower(a, ulo, uhi, kp);
        }
    }
    constexpr int kMaxRounds = 8;                  // T <= 256 probes, 32 per round
    const int nround = (T + 31) >> 5;
    int64_t bj[kMaxRounds];
#pragma unroll
    for (int t = 0; t < kMaxRounds; ++t) {
        bj[t] = -1;
        const int j = lane + 32 * t;
        if (t >= nround) continue;
        const int r = j % R, m = j / R;
        int64_t pr = p0;
        for (int rr = 1; rr < R; ++rr) {           // the lane holding key rr: rank rr - 1
            const unsigned hold = __ballot_sync(BLSH_FULL, lane < M && rank == rr - 1);
            const int64_t v = __shfl_sync(BLSH_FULL, pmine, __ffs(hold) - 1);
            if (r == rr) pr = v;
        }
        const int64_t off = (m & 1) ? -(int64_t)((m + 1) >> 1) : (int64_t)(m >> 1);
        const int64_t b = pr + off;
        if (j < T && b >= ulo && b < uhi) bj[t] = b;
    }
    // a bucket probed before is an empty probe: compare with every earlier in-range probe
    bool dup[kMaxRounds];
#pragma unroll
    for (int t = 0; t < kMaxRounds; ++t) dup[t] = false;
    if (R > 1) {
#pragma unroll
        for (int tt = 0; tt < kMaxRounds; ++tt) {
            if (tt >= nround) break;
            for (int sl = 0; sl < 32; ++sl) {
                const int64_t v = __shfl_sync(BLSH_FULL, bj[tt], sl);
                const int jj = sl + 32 * tt;
#pragma unroll
                for (int t = 0; t < kMaxRounds; ++t)
                    if (v >= 0 && v == bj[t] && jj < lane + 32 * t) dup[t] = true;
            }
        }
    }
    int64_t mysum = 0;
#pragma unroll
    for (int t = 0; t < kMaxRounds; ++t) {
        const int p = lane + 32 * t;
        if (t >= nround || p >= T) continue;
        const int64_t b = bj[t];
        const bool valid = b >= 0 && !dup[t];
        uint2 iv = make_uint2(0, 0);
        Key128 kb{0, 0};
        if (valid) {
            iv = make_uint2(a.uoff[b], a.uoff[b + 1]);
            kb = a.ukey[b];
        }
        ivl[p] = iv;
        mysum += (int64_t)(iv.y - iv.x);
        if (a.pkey) {
            a.pkey[(size_t)q * T + p] = kb;
            a.pvalid[(size_t)q * T + p] = valid ? 1 : 0;
        }
    }
    return mysum;
}

// T = 1 (standard probing): one thread per query -- the home key (the
// clamped home key equals the probe key whenever the code is in range) and
// one binary search; same outputs as k_probe_lookup.
__global__ void __launch_bounds__(256) k_lookup_home(QueryArgs a) {
    const int64_t q = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    if (q >= a.nq) return;
    const int oor = a.qoor[q];
    uint2* ivl = a.ivl + (size_t)q * 2;
    uint2 iv = make_uint2(0, 0);
    Key128 k{0, 0};
    const bool valid = !(oor & 7);
    if (valid) {
        const int g = a.qleaf[q];
        k = a.qkey[q];
        const int64_t u = find_bucket(a.ukey, a.leaf_u[g], a.leaf_u[g + 1], k);
        if (u >= 0) iv = make_uint2(a.uoff[u], a.uoff[u + 1]);
    }
    ivl[0] = iv;
    ivl[1] = make_uint2(0, 0);
    if (a.pkey) {
        a.pkey[q] = (oor & 2) ? Key128{0, 0} : k;
        a.pvalid[q] = valid ? 1 : 0;
    }
    const int64_t c = (int64_t)(iv.y - iv.x);
    a.base[q] = c;
    a.cnt[q] = c;
    if (a.level) a.level[q] = 0;
}

__global__ void __launch_bounds__(kPW * 32, 4) k_probe_lookup(QueryArgs a) {
    __shared__ ProbeSmem smem[kPW];
    const int lane = threadIdx.x & 31;
    const int w = threadIdx.x >> 5;
    const int64_t q = blockIdx.x * (int64_t)kPW + w;
    if (q >= a.nq) return;
    ProbeSmem& sm = smem[w];
    const int T = a.T;
    const int oor = a.qoor[q];
    uint2* ivl = a.ivl + (size_t)q * (T + 1);
    if (oor & 6) {   // leaf not owned by this shard, or a non-finite projection (R30): no probes
        for (int p = lane; p <= T; p += 32) ivl[p] = make_uint2(0, 0);
        if (a.pkey)
            for (int p = lane; p < T; p += 32) { a.pkey[(size_t)q * T + p] = Key128{0, 0}; a.pvalid[(size_t)q * T + p] = 0; }
        if (lane == 0) { a.base[q] = 0; a.cnt[q] = 0; if (a.level) a.level[q] = 0; }
        return;
    }
    const int g = a.qleaf[q];
    const int64_t ulo = a.leaf_u[g], uhi = a.leaf_u[g + 1];
    int64_t mysum = 0;
    if (a.probe == 3) {
        mysum = probe_curve(a, q, lane, ulo, uhi, ivl);
    } else if (a.quantizer == 1) {
        mysum = probe_e8(a, sm, q, lane, oor, ulo, uhi, ivl);
    } else {
        switch (a.M) {
#define BLSH_ZM_CASE(MMV) case MMV: mysum = probe_zm<MMV>(a, sm, q, lane, ulo, uhi, ivl); break;
            BLSH_ZM_CASE(1) BLSH_ZM_CASE(2) BLSH_ZM_CASE(3) BLSH_ZM_CASE(4) BLSH_ZM_CASE(5) BLSH_ZM_CASE(6)
            BLSH_ZM_CASE(7) BLSH_ZM_CASE(8) BLSH_ZM_CASE(9) BLSH_ZM_CASE(10) BLSH_ZM_CASE(11) BLSH_ZM_CASE(12)
            BLSH_ZM_CASE(13) BLSH_ZM_CASE(14) BLSH_ZM_CASE(15) BLSH_ZM_CASE(16)
#undef BLSH_ZM_CASE
            default: break;
        }
    }
    if (lane == 0) ivl[T] = make_uint2(0, 0);
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) mysum += __shfl_xor_sync(BLSH_FULL, mysum, o);
    if (lane == 0) {
        a.base[q] = mysum;
        a.cnt[q] = mysum;
        if (a.level) a.level[q] = 0;
    }
}
