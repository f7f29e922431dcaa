/*
 * oracle/blsh_oracle.c -- CPU ORACLE FOR BI-LEVEL LSH.  TEST INFRASTRUCTURE ONLY.
 *
 * Plain, slow, obviously-correct C implementation of what the query hot path
 * of Bi-level LSH (Pan & Manocha, ICDE 2012) computes.  Only tests/,
 * __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference legs
 * may load or call this library.  It shares no code, header, table or
 * constant generator with the CUDA product in paper_conf_icde_panm12_b200/;
 * both follow the readings written down in DESIGN.md ("Readings").
 *
 * Citations: "P:n" = line n of the paper text (/root/reference/PAPER.md, not
 * present at run time), with the section / equation it falls in.  "Rn" = the
 * numbered reading in DESIGN.md where the paper is silent or garbled.
 *
 * Compile with:  gcc -O2 -std=c11 -ffp-contract=off -fno-fast-math -fopenmp
 *                    -shared -fPIC -o liboracle.so blsh_oracle.c -lm
 * -ffp-contract=off guarantees that every a*b+c below is two roundings unless
 * written as an explicit fma()/fmaf() (R1).
 *
 * Parity status: every function is pinned by a -m "not gpu" test in tests/
 * (see DESIGN.md "Oracle pins"); none is "parity unpinned".
 */
#define _GNU_SOURCE
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <stdio.h>
#ifdef _OPENMP
#include <omp.h>
#endif

typedef unsigned __int128 u128;

#define ORC_E8_LEVELS 32   /* levels of the E8 code hierarchy searched (R27) */

/* ------------------------------------------------------------------------ */
/* R2: counter-based SplitMix64 generator.  P:43 draws a_i ~ N(0,1) and       */
/* b_i ~ U[0,W); P:98 draws a random unit direction per RP-tree node.  The   */
/* paper fixes no generator; R2 fixes this one so that the oracle and the    */
/* library can each implement it independently.                              */
/* ------------------------------------------------------------------------ */
static uint64_t orc_mix64(uint64_t z)
{
    z ^= z >> 30;
    z *= 0xBF58476D1CE4E5B9ULL;
    z ^= z >> 27;
    z *= 0x94D049BB133111EBULL;
    z ^= z >> 31;
    return z;
}

uint64_t orc_rng_u64(uint64_t seed, uint64_t stream, uint64_t i)
{
    return orc_mix64(seed + 0x9E3779B97F4A7C15ULL * ((stream << 32) + i + 1ULL));
}

/* U(stream, i) in [0,1) with 53 random bits (R2). */
double orc_rng_uniform(uint64_t seed, uint64_t stream, uint64_t i)
{
    return (double)(orc_rng_u64(seed, stream, i) >> 11) * 0x1.0p-53;
}

/* N(0,1) element i of a stream: Box-Muller, cosine branch only (R2). */
double orc_rng_gauss(uint64_t seed, uint64_t stream, uint64_t i)
{
    double u1 = orc_rng_uniform(seed, stream, 2 * i);
    double u2 = orc_rng_uniform(seed, stream, 2 * i + 1);
    return sqrt(-2.0 * log(1.0 - u1)) * cos(2.0 * 3.141592653589793 * u2);
}

static uint64_t orc_stream(uint64_t kind, uint64_t table, uint64_t idx)
{
    return (kind << 24) + (table << 16) + idx;
}

/* b1: per-leaf LSH parameters (Eq. 2; independent per leaf, P:84-86,
 * P:107, reading R3) and per-node RP directions.
 *   A[g][i][j] = fp32(N(0,1))        stream (1, 0, g), element i*d+j
 *   b[g][i]    = fp32(W_g * U[0,1))  stream (2, 0, g), element i; clamped < W_g
 *   dir[v][j]  = fp32(g_j / |g|)     stream (3, 0, v), fp64 normalisation
 *   jit[v]     = U[0,1)              stream (4, 0, v), element 0 (max rule)  */
/* The L hash tables of P:43 ("L hash tables are used and each of them is
 * constructed independently with different dim-M hash functions") get their
 * own (a, b) per leaf: table l draws from streams (1, l, g) and (2, l, g)
 * (R2, R24).  Table 0 is the single table of the L = 1 index. */
void orc_gen_table_params(uint64_t seed, int table, int G, int M, int d, const float *Wleaf,
                          float *A, float *b)
{
    for (int g = 0; g < G; g++) {
        for (int i = 0; i < M; i++)
            for (int j = 0; j < d; j++)
                A[((size_t)g * M + i) * d + j] =
                    (float)orc_rng_gauss(seed, orc_stream(1, (uint64_t)table, g), (uint64_t)i * d + j);
        for (int i = 0; i < M; i++) {
            float W = Wleaf[g];
            double u = orc_rng_uniform(seed, orc_stream(2, (uint64_t)table, g), i);
            float bf = (float)((double)W * u);
            if (bf >= W) bf = nextafterf(W, 0.0f);      /* R2: keep b in [0, W) */
            b[(size_t)g * M + i] = bf;
        }
    }
}

void orc_gen_params(uint64_t seed, int G, int M, int d, const float *Wleaf,
                    float *A, float *b, float *dirs, double *jit)
{
    orc_gen_table_params(seed, 0, G, M, d, Wleaf, A, b);
    double *gv = (double *)malloc(sizeof(double) * (size_t)d);
    for (int v = 0; v < G - 1; v++) {
        double s = 0.0;
        for (int j = 0; j < d; j++) {
            gv[j] = orc_rng_gauss(seed, orc_stream(3, 0, v), j);
            s = fma(gv[j], gv[j], s);
        }
        double nrm = sqrt(s);
        for (int j = 0; j < d; j++) dirs[(size_t)v * d + j] = (float)(gv[j] / nrm);
        jit[v] = orc_rng_uniform(seed, orc_stream(4, 0, v), 0);
    }
    free(gv);
}

/* ------------------------------------------------------------------------ */
/* R1: canonical fp32 arithmetic.  Strict ascending-j fma chains.            */
/* ------------------------------------------------------------------------ */
static float orc_dotc(const float *a, const float *x, int d)
{
    float s = 0.0f;
    for (int j = 0; j < d; j++) s = fmaf(a[j], x[j], s);
    return s;
}

static float orc_dist2c(const float *x, const float *y, int d)
{
    float s = 0.0f;
    for (int j = 0; j < d; j++) {
        float e = x[j] - y[j];
        s = fmaf(e, e, s);
    }
    return s;
}

float orc_dot_canonical(const float *a, const float *x, int d) { return orc_dotc(a, x, d); }
float orc_dist2_canonical(const float *x, const float *y, int d) { return orc_dist2c(x, y, d); }

/* Total order on fp32 values used for the median (R5). */
static uint32_t orc_fkey(float f)
{
    uint32_t u;
    memcpy(&u, &f, 4);
    return (u & 0x80000000u) ? ~u : (u | 0x80000000u);
}

static float orc_fkey_inv(uint32_t k)
{
    uint32_t u = (k & 0x80000000u) ? (k & 0x7FFFFFFFu) : ~k;
    float f;
    memcpy(&f, &u, 4);
    return f;
}

/* ------------------------------------------------------------------------ */
/* Morton code of an LSH code (Sec. IV-B2a; bit layout reading R9).   */
/* u_i = code_i + 2^(B-1);  key bit (p*M + (M-1-i)) = bit p of u_i.          */
/* ------------------------------------------------------------------------ */
int orc_bits_per_coord(int M)
{
    int B = 128 / M;
    return B > 24 ? 24 : B;
}

static u128 orc_morton(const int32_t *code, int M, int B)
{
    u128 key = 0;
    for (int p = B - 1; p >= 0; p--)
        for (int i = 0; i < M; i++) {
            uint32_t u = (uint32_t)(code[i] + (1 << (B - 1)));
            u128 bit = (u >> p) & 1u;
            key |= bit << (p * M + (M - 1 - i));
        }
    return key;
}

void orc_morton_encode(const int32_t *code, int M, uint64_t *hi, uint64_t *lo)
{
    u128 k = orc_morton(code, M, orc_bits_per_coord(M));
    *hi = (uint64_t)(k >> 64);
    *lo = (uint64_t)k;
}

void orc_morton_decode(uint64_t hi, uint64_t lo, int M, int32_t *code)
{
    int B = orc_bits_per_coord(M);
    u128 k = ((u128)hi << 64) | lo;
    for (int i = 0; i < M; i++) {
        uint32_t u = 0;
        for (int p = 0; p < B; p++)
            u |= (uint32_t)((k >> (p * M + (M - 1 - i))) & 1u) << p;
        code[i] = (int32_t)u - (1 << (B - 1));
    }
}

static int orc_code_in_range(const int32_t *code, int M, int B)
{
    for (int i = 0; i < M; i++)
        if (code[i] < -(1 << (B - 1)) || code[i] > (1 << (B - 1)) - 1) return 0;
    return 1;
}

/* ------------------------------------------------------------------------ */
/* E8 decoder (Eq. 6; tie-breaks reading R14).                    */
/* Output in doubled coordinates c2 = 2c (even for D8, odd for D8 + 1/2).   */
/* ------------------------------------------------------------------------ */
static void orc_d8_nearest(const float *w, int32_t *z)
{
    /* nearest point of D8 (integer vectors with even sum) to w */
    int32_t sum = 0;
    for (int j = 0; j < 8; j++) {
        z[j] = (int32_t)rintf(w[j]);                 /* round half to even */
        sum += z[j];
    }
    if (sum & 1) {
        int jb = 0;
        float best = -1.0f;
        for (int j = 0; j < 8; j++) {
            float dev = fabsf(w[j] - (float)z[j]);
            if (dev > best) { best = dev; jb = j; }   /* ties -> lowest j */
        }
        float r = w[jb] - (float)z[jb];
        z[jb] += (r >= 0.0f) ? 1 : -1;                /* 0 -> +1 */
    }
}

static double orc_e8_dist2(const float *y, const int32_t *c2)
{
    double s = 0.0;
    for (int j = 0; j < 8; j++) {
        double e = (double)y[j] - 0.5 * (double)c2[j];
        s = fma(e, e, s);
    }
    return s;
}

void orc_e8_decode(const float *y, int32_t *c2)
{
    int32_t z0[8], z1[8], a[8], b[8];
    float w[8];
    orc_d8_nearest(y, z0);
    for (int j = 0; j < 8; j++) w[j] = y[j] - 0.5f;
    orc_d8_nearest(w, z1);
    for (int j = 0; j < 8; j++) { a[j] = 2 * z0[j]; b[j] = 2 * z1[j] + 1; }
    double d0 = orc_e8_dist2(y, a), d1 = orc_e8_dist2(y, b);
    if (d1 < d0) memcpy(c2, b, sizeof b);              /* ties -> integer coset */
    else memcpy(c2, a, sizeof a);
}

/* E8 hierarchy (Eq. 10; reading R27): the parent of an E8 code is
 * DECODE of half of it, so in doubled coordinates c = 2p the parent code is
 * DECODE(c / 4) (exact in fp32 for |c| < 2^24).  Level-j code of a bucket or
 * query = the parent applied j times to its level-0 code. */
void orc_e8_parent(const int32_t *c2, int32_t *out)
{
    float y[8];
    for (int i = 0; i < 8; i++) y[i] = (float)c2[i] * 0.25f;
    orc_e8_decode(y, out);
}

/* The 240 minimal vectors of E8 in canonical order (R15), doubled coords. */
void orc_e8_roots(int32_t *roots /* [240][8] */)
{
    int r = 0;
    for (int i = 0; i < 8; i++)
        for (int j = i + 1; j < 8; j++)
            for (int si = 0; si < 2; si++)
                for (int sj = 0; sj < 2; sj++) {
                    for (int t = 0; t < 8; t++) roots[r * 8 + t] = 0;
                    roots[r * 8 + i] = si ? -2 : 2;
                    roots[r * 8 + j] = sj ? -2 : 2;
                    r++;
                }
    for (int mask = 0; mask < 256; mask++) {
        if (__builtin_popcount(mask) & 1) continue;
        for (int t = 0; t < 8; t++) roots[r * 8 + t] = ((mask >> t) & 1) ? -1 : 1;
        r++;
    }
}

/* ------------------------------------------------------------------------ */
/* Multiprobe sequence ("heap-based method in [8]"; reading R11) */
/* Defined by full enumeration: all delta in {-1,0,1}^M \ {0}, ordered by     */
/* (score, enc); score = sum over perturbed i (ascending) of x_i(delta_i)^2 */
/* in fp64 with x_i(-1) = t_i - h_i, x_i(+1) = 1 - x_i(-1) (fp32).           */
/* ------------------------------------------------------------------------ */
typedef struct { double score; int32_t enc; } orc_probe;

static int orc_probe_cmp(const void *pa, const void *pb)
{
    const orc_probe *a = (const orc_probe *)pa, *b = (const orc_probe *)pb;
    if (a->score < b->score) return -1;
    if (a->score > b->score) return 1;
    return (a->enc > b->enc) - (a->enc < b->enc);
}

static int32_t orc_pow3(int M) { int32_t p = 1; for (int i = 0; i < M; i++) p *= 3; return p; }

/* deltas: [(T-1) x M] perturbation vectors after the home bucket, for the
 * unclamped floor codes f_i = floor(t_i). */
int orc_multiprobe_deltas(const float *t, int M, int T, int32_t *deltas, double *scores)
{
    if (M > 10 || T < 1) return -1;
    int32_t P = orc_pow3(M);
    if (T > P) return -1;
    float xm[16], xp[16];
    for (int i = 0; i < M; i++) {
        xm[i] = t[i] - floorf(t[i]);
        xp[i] = 1.0f - xm[i];
    }
    orc_probe *all = (orc_probe *)malloc(sizeof(orc_probe) * (size_t)P);
    int32_t home = 0;
    for (int i = 0; i < M; i++) home = home * 3 + 1;
    int np = 0;
    for (int32_t enc = 0; enc < P; enc++) {
        if (enc == home) continue;
        double s = 0.0;
        int32_t e = enc;
        int dig[16];
        for (int i = M - 1; i >= 0; i--) { dig[i] = e % 3; e /= 3; }
        for (int i = 0; i < M; i++) {
            if (dig[i] == 0) s += (double)xm[i] * (double)xm[i];
            else if (dig[i] == 2) s += (double)xp[i] * (double)xp[i];
        }
        all[np].score = s;
        all[np].enc = enc;
        np++;
    }
    qsort(all, (size_t)np, sizeof(orc_probe), orc_probe_cmp);
    for (int r = 0; r < T - 1; r++) {
        int32_t e = all[r].enc;
        for (int i = M - 1; i >= 0; i--) { deltas[r * M + i] = (e % 3) - 1; e /= 3; }
        if (scores) scores[r] = all[r].score;
    }
    free(all);
    return 0;
}

/* Lattice probe order (R15): the 240 neighbours c + r of the  */
/* home E8 point c, ordered by (fp64 |y - c - r|^2, root index).            */
/* Recursive E8 probing ("If the number of candidates computed is not
 * enough, we recursively probe the adjacent buckets of the 240 probed
 * buckets"; reading R26): the second ring S2 = {r + r'} minus {0} and the roots
 * = the E8 vectors of norm^2 4 (2160), 6 (6720) and 8 (the 240 vectors 2r),
 * in doubled coordinates, ordered by (norm^2, coordinates lexicographically as
 * signed integers).  Probes 242.. of a lattice sequence take them by
 * (distance to the query, this order). */
#define ORC_E8_S2 9120
static int orc_vec8_cmp(const void *pa, const void *pb)
{
    const int32_t *a = (const int32_t *)pa, *b = (const int32_t *)pb;
    int32_t na = 0, nb = 0;
    for (int j = 0; j < 8; j++) { na += a[j] * a[j]; nb += b[j] * b[j]; }
    if (na != nb) return na < nb ? -1 : 1;
    for (int j = 0; j < 8; j++) if (a[j] != b[j]) return a[j] < b[j] ? -1 : 1;
    return 0;
}

int orc_e8_second_ring(int32_t *out /* [ORC_E8_S2][8] */)
{
    int32_t roots[240 * 8];
    orc_e8_roots(roots);
    int32_t *all = (int32_t *)malloc(sizeof(int32_t) * 8 * 240 * 240);
    int m = 0;
    for (int r = 0; r < 240; r++)
        for (int q = 0; q < 240; q++) {
            int32_t v[8], n2 = 0;
            for (int j = 0; j < 8; j++) { v[j] = roots[r * 8 + j] + roots[q * 8 + j]; n2 += v[j] * v[j]; }
            if (n2 < 16) continue;              /* 0 (r' = -r) and the roots themselves (norm^2 2 = 8 doubled) */
            memcpy(all + 8 * m, v, sizeof(v));
            m++;
        }
    qsort(all, (size_t)m, sizeof(int32_t) * 8, orc_vec8_cmp);
    int u = 0;
    for (int i = 0; i < m; i++)
        if (u == 0 || orc_vec8_cmp(all + 8 * i, out + 8 * (u - 1)) != 0) {
            if (u < ORC_E8_S2) memcpy(out + 8 * u, all + 8 * i, sizeof(int32_t) * 8);
            u++;
        }
    free(all);
    return u;
}

int orc_lattice_order(const float *y, const int32_t *c2, int T, int32_t *root_idx);

/* Lattice probing with M = 16 (two E8 blocks, R28): the neighbours of the
 * home code c change one block by one root; candidate x = blk * 240 + r,
 * ordered by (fp64 sum over all M coordinates of (y_j - c'_j / 2)^2, x). */
static double orc_e8_dist2_m(const float *y, const int32_t *c2, int M)
{
    double s = 0.0;
    for (int j = 0; j < M; j++) {
        double e = (double)y[j] - 0.5 * (double)c2[j];
        s = fma(e, e, s);
    }
    return s;
}

int orc_lattice_order_blocks(const float *y, const int32_t *c2, int M, int T, int32_t *idx)
{
    if (M == 8) return orc_lattice_order(y, c2, T, idx);
    const int P = 240 * (M / 8);
    if (T < 1 || T > 1 + P || T > 256) return -1;
    int32_t roots[240 * 8];
    orc_e8_roots(roots);
    orc_probe *all = (orc_probe *)malloc(sizeof(orc_probe) * (size_t)P);
    for (int x = 0; x < P; x++) {
        int32_t p[16];
        memcpy(p, c2, sizeof(int32_t) * M);
        for (int j = 0; j < 8; j++) p[8 * (x / 240) + j] += roots[(x % 240) * 8 + j];
        all[x].score = orc_e8_dist2_m(y, p, M);
        all[x].enc = x;
    }
    qsort(all, (size_t)P, sizeof(orc_probe), orc_probe_cmp);
    for (int r = 0; r < T - 1; r++) idx[r] = all[r].enc;
    free(all);
    return 0;
}

int orc_lattice_order(const float *y, const int32_t *c2, int T, int32_t *root_idx)
{
    if (T < 1 || T > 256) return -1;
    int32_t roots[240 * 8];
    orc_e8_roots(roots);
    orc_probe all[240];
    for (int r = 0; r < 240; r++) {
        int32_t p[8];
        for (int j = 0; j < 8; j++) p[j] = c2[j] + roots[r * 8 + j];
        all[r].score = orc_e8_dist2(y, p);
        all[r].enc = r;
    }
    qsort(all, 240, sizeof(orc_probe), orc_probe_cmp);
    for (int r = 0; r < T - 1 && r < 240; r++) root_idx[r] = all[r].enc;
    if (T > 241) {           /* recursive probing: the second ring, index 240 + i */
        int32_t *s2 = (int32_t *)malloc(sizeof(int32_t) * 8 * ORC_E8_S2);
        orc_e8_second_ring(s2);
        orc_probe *ring = (orc_probe *)malloc(sizeof(orc_probe) * ORC_E8_S2);
        for (int i = 0; i < ORC_E8_S2; i++) {
            int32_t p[8];
            for (int j = 0; j < 8; j++) p[j] = c2[j] + s2[i * 8 + j];
            ring[i].score = orc_e8_dist2(y, p);
            ring[i].enc = i;
        }
        qsort(ring, ORC_E8_S2, sizeof(orc_probe), orc_probe_cmp);
        for (int r = 240; r < T - 1; r++) root_idx[r] = 240 + (int32_t)ring[r - 240].enc;
        free(ring);
        free(s2);
    }
    return 0;
}

/* ------------------------------------------------------------------------ */
/* Index                                                                     */
/* ------------------------------------------------------------------------ */
typedef struct {
    int64_t n;
    int d, G, M, quantizer, B, depth;
    int rp_rule;
    double rp_mean_c, rp_max_jitter;
    int ek_iters;
    const float *X;       /* borrowed, row-major n x d */
    float *Wl;            /* [G] */
    float *A, *b;         /* [G][M][d], [G][M] */
    float *dirs;          /* [G-1][d] */
    double *jit;          /* [G-1] */
    float *mu;            /* [G-1][d] node means (mean rule), 0 otherwise */
    float *theta;         /* [G-1] */
    int32_t *ntype;       /* [G-1] 0 = hyperplane, 1 = sphere */
    double *diam2, *da2;  /* [G-1] diagnostics of the mean-rule test */
    int32_t *leaf;        /* [n] */
    int32_t *code;        /* [n][M]: floor codes (Z^M) or doubled E8 codes */
    u128 *key;            /* [n] */
    int64_t *perm;        /* [n] table position -> original id */
    int64_t nu;           /* number of buckets */
    u128 *ukey;           /* [nu] */
    int32_t *uleaf;       /* [nu] */
    int64_t *uoff;        /* [nu+1] */
    int64_t *leaf_u;      /* [G+1] first bucket of each leaf */
    /* last query (stages for parity tests) */
    int64_t lq_n;
    int lq_T;
    int32_t *lq_leaf;     /* [nq] */
    float *lq_t;          /* [nq][M] */
    int32_t *lq_code;     /* [nq][M] */
    int32_t *lq_oor;      /* [nq] home code out of range */
    uint64_t *lq_key;     /* [nq][2] hi, lo */
    uint64_t *lq_pkey;    /* [nq][T][2] probe keys */
    int32_t *lq_pvalid;   /* [nq][T] */
    int64_t *lq_base;     /* [nq] |A0| */
    int32_t *lq_level;    /* [nq] key bits cleared by the hierarchy (0 = none) */
    int64_t lq_tau;
    int64_t *lq_coff;     /* [nq+1] */
    int64_t *lq_cand;     /* sorted candidate ids */
} orc_index;

static void orc_chunked_colsum(const float *X, int d, const int64_t *ids, int64_t n, double *tot)
{
    /* R7: ordered fp64 reduction per coordinate j; chunks of 4096 members
     * (ascending id), each summed sequentially, chunk sums added in chunk
     * order.  All coordinates are walked together row by row (the sequence
     * of additions of every single coordinate is unchanged). */
    int64_t nc = (n + 4095) / 4096;
    double *part = (double *)calloc((size_t)(nc > 0 ? nc : 1) * d, sizeof(double));
    #pragma omp parallel for schedule(dynamic, 1)
    for (int64_t c = 0; c < nc; c++) {
        double *p = part + (size_t)c * d;
        int64_t e = (c + 1) * 4096 < n ? (c + 1) * 4096 : n;
        for (int64_t i = c * 4096; i < e; i++) {
            const float *x = X + ids[i] * (int64_t)d;
            for (int j = 0; j < d; j++) p[j] += (double)x[j];
        }
    }
    for (int j = 0; j < d; j++) tot[j] = 0.0;
    for (int64_t c = 0; c < nc; c++)
        for (int j = 0; j < d; j++) tot[j] += part[(size_t)c * d + j];
    free(part);
}

static double orc_chunked_sum_vals(const float *v, int64_t n)
{
    double tot = 0.0;
    for (int64_t c = 0; c < n; c += 4096) {
        double p = 0.0;
        int64_t e = c + 4096 < n ? c + 4096 : n;
        for (int64_t i = c; i < e; i++) p += (double)v[i];
        tot += p;
    }
    return tot;
}

/* Approximate diameter (Egecioglu-Kalantari [22]; reading R6).   */
/* Returns the squared estimate: the largest canonical dist2 between any two */
/* of the m selected points.  sel_out (optional) receives the selected ids.  */
static float orc_diameter2(const float *X, int d, const int64_t *S, int64_t nS, int m_req,
                           int64_t *sel_out, float *r1sq)
{
    if (nS == 0) { if (r1sq) *r1sq = 0.0f; return 0.0f; }
    int m = m_req < nS ? m_req : (int)nS;
    if (m < 1) m = 1;
    int64_t *sel = (int64_t *)malloc(sizeof(int64_t) * (size_t)m);
    double *acc = (double *)calloc((size_t)nS, sizeof(double));
    float *dd = (float *)malloc(sizeof(float) * (size_t)nS);
    const float *p0 = X + S[0] * (int64_t)d;
    #pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < nS; i++) dd[i] = orc_dist2c(X + S[i] * (int64_t)d, p0, d);
    int64_t best = 0;
    for (int64_t i = 1; i < nS; i++) if (dd[i] > dd[best]) best = i;
    sel[0] = S[best];
    for (int it = 0; it + 1 < m; it++) {
        const float *xs = X + sel[it] * (int64_t)d;
        #pragma omp parallel for schedule(static)
        for (int64_t i = 0; i < nS; i++) acc[i] += (double)orc_dist2c(X + S[i] * (int64_t)d, xs, d);
        best = 0;
        for (int64_t i = 1; i < nS; i++) if (acc[i] > acc[best]) best = i;
        sel[it + 1] = S[best];
    }
    float mx = 0.0f;
    for (int a = 0; a < m; a++)
        for (int c = a + 1; c < m; c++) {
            float v = orc_dist2c(X + sel[a] * (int64_t)d, X + sel[c] * (int64_t)d, d);
            if (v > mx) mx = v;
        }
    if (r1sq) *r1sq = (m >= 2) ? orc_dist2c(X + sel[0] * (int64_t)d, X + sel[1] * (int64_t)d, d) : 0.0f;
    if (sel_out) memcpy(sel_out, sel, sizeof(int64_t) * (size_t)m);
    free(sel); free(acc); free(dd);
    return mx;
}

/* Exported for the diameter-bound test. */
float orc_diameter_estimate(const float *X, int d, const int64_t *S, int64_t nS, int m,
                            float *r1sq, int64_t *sel_out)
{
    return orc_diameter2(X, d, S, nS, m, sel_out, r1sq);
}

static int orc_cmp_u32(const void *a, const void *b)
{
    uint32_t x = *(const uint32_t *)a, y = *(const uint32_t *)b;
    return (x > y) - (x < y);
}

/* Split one RP-tree node (rules of [20] as read in R4-R7). */
static void orc_split_node(orc_index *ix, int v, const int64_t *S, int64_t nS, float *s_out)
{
    const int d = ix->d;
    const float *X = ix->X;
    float *mu = ix->mu + (size_t)v * d;
    ix->ntype[v] = 0;
    ix->diam2[v] = 0.0;
    ix->da2[v] = 0.0;
    if (nS == 0) { ix->theta[v] = 0.0f; return; }
    if (ix->rp_rule == 0) {
        /* RP-tree mean: mean, average squared interpoint distance
         * Delta_A^2 = (2/|S|) sum |x - mu|^2, approximate diameter Delta. */
        double *tot = (double *)malloc(sizeof(double) * (size_t)d);
        orc_chunked_colsum(X, d, S, nS, tot);
        for (int j = 0; j < d; j++) mu[j] = (float)(tot[j] / (double)nS);
        free(tot);
        float *e = (float *)malloc(sizeof(float) * (size_t)nS);
        #pragma omp parallel for schedule(static)
        for (int64_t i = 0; i < nS; i++) e[i] = orc_dist2c(X + S[i] * (int64_t)d, mu, d);
        double da2 = 2.0 * orc_chunked_sum_vals(e, nS) / (double)nS;
        free(e);
        float diam2 = orc_diameter2(X, d, S, nS, ix->ek_iters, NULL, NULL);
        ix->diam2[v] = (double)diam2;
        ix->da2[v] = da2;
        ix->ntype[v] = ((double)diam2 <= ix->rp_mean_c * da2) ? 0 : 1;
    }
    const float *dir = ix->dirs + (size_t)v * d;
    #pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < nS; i++)
        s_out[i] = ix->ntype[v] == 0 ? orc_dotc(dir, X + S[i] * (int64_t)d, d)
                                     : orc_dist2c(X + S[i] * (int64_t)d, mu, d);
    /* lower median (R5): rank floor((|S|-1)/2) in the total order */
    uint32_t *k = (uint32_t *)malloc(sizeof(uint32_t) * (size_t)nS);
    for (int64_t i = 0; i < nS; i++) k[i] = orc_fkey(s_out[i]);
    qsort(k, (size_t)nS, sizeof(uint32_t), orc_cmp_u32);
    float theta = orc_fkey_inv(k[(nS - 1) / 2]);
    free(k);
    if (ix->rp_rule == 1 && ix->rp_max_jitter != 0.0) {
        /* RP-tree max jitter [20] (R4): delta = (2u-1) * j * |x0 - y| / sqrt(d) */
        const float *x0 = X + S[0] * (int64_t)d;
        int64_t best = 0;
        float bd = -1.0f;
        for (int64_t i = 0; i < nS; i++) {
            float dv = orc_dist2c(X + S[i] * (int64_t)d, x0, d);
            if (dv > bd) { bd = dv; best = i; }
        }
        (void)best;
        double delta = (2.0 * ix->jit[v] - 1.0) * ix->rp_max_jitter * sqrt((double)bd) /
                       sqrt((double)d);
        theta = (float)((double)theta + delta);
    }
    ix->theta[v] = theta;
}

static void orc_free_lastq(orc_index *ix)
{
    free(ix->lq_leaf); free(ix->lq_t); free(ix->lq_code); free(ix->lq_oor); free(ix->lq_key);
    free(ix->lq_pkey); free(ix->lq_pvalid); free(ix->lq_base); free(ix->lq_level);
    free(ix->lq_coff); free(ix->lq_cand);
    ix->lq_leaf = NULL; ix->lq_t = NULL; ix->lq_code = NULL; ix->lq_oor = NULL; ix->lq_key = NULL;
    ix->lq_pkey = NULL; ix->lq_pvalid = NULL; ix->lq_base = NULL; ix->lq_level = NULL;
    ix->lq_coff = NULL; ix->lq_cand = NULL;
    ix->lq_n = 0;
}

void orc_free(orc_index *ix)
{
    if (!ix) return;
    free(ix->Wl); free(ix->A); free(ix->b); free(ix->dirs); free(ix->jit); free(ix->mu);
    free(ix->theta); free(ix->ntype); free(ix->diam2); free(ix->da2); free(ix->leaf);
    free(ix->code); free(ix->key); free(ix->perm); free(ix->ukey); free(ix->uleaf);
    free(ix->uoff); free(ix->leaf_u);
    orc_free_lastq(ix);
    free(ix);
}

/* Hash one vector with leaf g's parameters (Eq. 2; Eq. 6).     */
/* Returns 1 if the code is inside the B-bit Morton range.                  */
static int orc_hash(const orc_index *ix, int g, const float *x, float *t, int32_t *code,
                    int32_t *clamped)
{
    const int M = ix->M, d = ix->d, B = ix->B;
    const float W = ix->Wl[g];
    for (int i = 0; i < M; i++) {
        float dot = orc_dotc(ix->A + ((size_t)g * M + i) * d, x, d);
        float num = dot + ix->b[(size_t)g * M + i];
        t[i] = num / W;
    }
    const float lo = -(float)(1 << (B - 1)), hi = (float)((1 << (B - 1)) - 1);
    int ok = 1;
    if (ix->quantizer == 0) {
        for (int i = 0; i < M; i++) {
            float f = floorf(t[i]);
            float c = f < lo ? lo : (f > hi ? hi : f);
            if (c != f) ok = 0;
            code[i] = (int32_t)c;
            if (clamped) clamped[i] = (int32_t)c;
        }
    } else {
        /* E8 (Eq. 6); M = 16: two E8 blocks decoded independently (R28) */
        for (int i = 0; i < M; i++)
            if (!(fabsf(t[i]) < 16000.0f)) ok = 0;
        if (ok) {
            for (int blk = 0; blk < M / 8; blk++) orc_e8_decode(t + 8 * blk, code + 8 * blk);
            if (!orc_code_in_range(code, M, B)) ok = 0;
        }
        if (!ok) for (int i = 0; i < M; i++) code[i] = 0;
        if (clamped) memcpy(clamped, code, sizeof(int32_t) * M);
    }
    return ok;
}

/* Eq. 2 for one vector with explicit parameters (used by the collision-
 * probability and closed-form tests): t_i = (a_i . x + b_i) / W, h_i = floor. */
void orc_hash_point(const float *A, const float *b, float W, int M, int d, const float *x,
                    float *t, int32_t *h)
{
    for (int i = 0; i < M; i++) {
        float dot = orc_dotc(A + (size_t)i * d, x, d);
        float num = dot + b[i];
        t[i] = num / W;
        h[i] = (int32_t)floorf(t[i]);
    }
}

static int orc_route(const orc_index *ix, const float *x)
{
    int v = 0;
    for (int l = 0; l < ix->depth; l++) {
        float s = ix->ntype[v] == 0 ? orc_dotc(ix->dirs + (size_t)v * ix->d, x, ix->d)
                                    : orc_dist2c(x, ix->mu + (size_t)v * ix->d, ix->d);
        v = 2 * v + 1 + (s > ix->theta[v] ? 1 : 0);
    }
    return v - (ix->G - 1);
}

typedef struct { int32_t leaf; u128 key; int64_t id; } orc_entry;

static int orc_entry_cmp(const void *pa, const void *pb)
{
    const orc_entry *a = (const orc_entry *)pa, *b = (const orc_entry *)pb;
    if (a->leaf != b->leaf) return a->leaf < b->leaf ? -1 : 1;
    if (a->key != b->key) return a->key < b->key ? -1 : 1;
    return (a->id > b->id) - (a->id < b->id);
}

/* Build: b1 params, b2 RP-tree, b3 hash, b4 table.  Returns NULL and sets
 * *err: 1 invalid argument, 4 code outside the Morton range (R9). */
orc_index *orc_build(const float *X, int64_t n, int d, int G, int M, int quantizer, float W,
                     const float *Wleaf, int rp_rule, double rp_mean_c, double rp_max_jitter,
                     int ek_iters, uint64_t seed, int table, int W_rule, int *err)
{
    *err = 1;
    if (n < 0 || d < 1 || G < 1 || G > 4096 || (G & (G - 1)) || M < 1 || M > 16) return NULL;
    if (table < 0 || table > 255) return NULL;
    if (W_rule != 0 && W_rule != 1) return NULL;
    if (W_rule == 1 && Wleaf) return NULL;
    if (quantizer == 1 && M != 8 && M != 16) return NULL;   /* ceil(M/8) E8 blocks, R28 */
    if (!(W > 0.0f)) return NULL;
    orc_index *ix = (orc_index *)calloc(1, sizeof(orc_index));
    ix->n = n; ix->d = d; ix->G = G; ix->M = M; ix->quantizer = quantizer;
    ix->B = orc_bits_per_coord(M);
    ix->rp_rule = rp_rule; ix->rp_mean_c = rp_mean_c; ix->rp_max_jitter = rp_max_jitter;
    ix->ek_iters = ek_iters;
    ix->X = X;
    int depth = 0;
    while ((1 << depth) < G) depth++;
    ix->depth = depth;
    int nn = G - 1 > 0 ? G - 1 : 1;
    ix->Wl = (float *)malloc(sizeof(float) * G);
    for (int g = 0; g < G; g++) ix->Wl[g] = Wleaf ? Wleaf[g] : W;
    for (int g = 0; g < G; g++) if (!(ix->Wl[g] > 0.0f)) { orc_free(ix); return NULL; }
    ix->A = (float *)malloc(sizeof(float) * (size_t)G * M * d);
    ix->b = (float *)malloc(sizeof(float) * (size_t)G * M);
    ix->dirs = (float *)calloc((size_t)nn * d, sizeof(float));
    ix->jit = (double *)calloc((size_t)nn, sizeof(double));
    ix->mu = (float *)calloc((size_t)nn * d, sizeof(float));
    ix->theta = (float *)calloc((size_t)nn, sizeof(float));
    ix->ntype = (int32_t *)calloc((size_t)nn, sizeof(int32_t));
    ix->diam2 = (double *)calloc((size_t)nn, sizeof(double));
    ix->da2 = (double *)calloc((size_t)nn, sizeof(double));
    orc_gen_params(seed, G, M, d, ix->Wl, ix->A, ix->b, ix->dirs, ix->jit);
    /* table l of an L-table index: same RP-tree (dirs, jit), its own (a, b) */
    if (table > 0) orc_gen_table_params(seed, table, G, M, d, ix->Wl, ix->A, ix->b);

    /* b2: level-by-level RP-tree; members of each node kept in ascending id. */
    int64_t *order = (int64_t *)malloc(sizeof(int64_t) * (size_t)(n > 0 ? n : 1));
    int64_t *tmp = (int64_t *)malloc(sizeof(int64_t) * (size_t)(n > 0 ? n : 1));
    float *s = (float *)malloc(sizeof(float) * (size_t)(n > 0 ? n : 1));
    int64_t *seg = (int64_t *)calloc((size_t)G + 1, sizeof(int64_t));
    int64_t *nseg = (int64_t *)calloc((size_t)G + 1, sizeof(int64_t));
    for (int64_t i = 0; i < n; i++) order[i] = i;
    seg[0] = 0; seg[1] = n;
    for (int l = 0; l < depth; l++) {
        int nodes = 1 << l;
        for (int k = 0; k < nodes; k++) {
            int v = (nodes - 1) + k;
            int64_t a = seg[k], e = seg[k + 1];
            orc_split_node(ix, v, order + a, e - a, s);
            int64_t nl = 0, p = a;
            for (int64_t i = a; i < e; i++) if (s[i - a] <= ix->theta[v]) { tmp[p++] = order[i]; nl++; }
            for (int64_t i = a; i < e; i++) if (!(s[i - a] <= ix->theta[v])) tmp[p++] = order[i];
            nseg[2 * k] = a;
            nseg[2 * k + 1] = a + nl;
        }
        nseg[2 * nodes] = n;
        memcpy(order, tmp, sizeof(int64_t) * (size_t)n);
        memcpy(seg, nseg, sizeof(int64_t) * ((size_t)2 * nodes + 1));
    }
    ix->leaf = (int32_t *)malloc(sizeof(int32_t) * (size_t)(n > 0 ? n : 1));
    for (int g = 0; g < G; g++)
        for (int64_t i = seg[g]; i < seg[g + 1]; i++) ix->leaf[order[i]] = g;

    /* P:107 "different LSH parameters (e.g. bucket size W) ... for each cell"
     * (R29): W_g = fp32(W sqrt(D_g / D_med)), D_g = Delta_A^2 of leaf g with
     * the R7 reductions (members in ascending id), D_med = lower median of the
     * D_g; W_g = W when D_g = 0.  (a, b) are redrawn with the new widths. */
    if (W_rule == 1) {
        double *D = (double *)calloc((size_t)G, sizeof(double));
        double *tot = (double *)malloc(sizeof(double) * (size_t)d);
        float *mu = (float *)malloc(sizeof(float) * (size_t)d);
        for (int g = 0; g < G; g++) {
            int64_t nS = seg[g + 1] - seg[g];
            if (nS == 0) continue;
            const int64_t *S = order + seg[g];
            orc_chunked_colsum(X, d, S, nS, tot);
            for (int j = 0; j < d; j++) mu[j] = (float)(tot[j] / (double)nS);
            float *e = (float *)malloc(sizeof(float) * (size_t)nS);
            for (int64_t i = 0; i < nS; i++) e[i] = orc_dist2c(X + S[i] * (int64_t)d, mu, d);
            D[g] = 2.0 * orc_chunked_sum_vals(e, nS) / (double)nS;
            free(e);
        }
        double *srt = (double *)malloc(sizeof(double) * (size_t)G);
        memcpy(srt, D, sizeof(double) * (size_t)G);
        for (int a = 1; a < G; a++) {          /* insertion sort: G <= 4096 */
            double v = srt[a];
            int b = a - 1;
            while (b >= 0 && srt[b] > v) { srt[b + 1] = srt[b]; b--; }
            srt[b + 1] = v;
        }
        double med = srt[(G - 1) / 2];
        for (int g = 0; g < G; g++) {
            float wg = (D[g] > 0.0 && med > 0.0) ? (float)((double)W * sqrt(D[g] / med)) : W;
            if (!(wg > 0.0f) || !isfinite(wg)) wg = W;
            ix->Wl[g] = wg;
        }
        orc_gen_params(seed, G, M, d, ix->Wl, ix->A, ix->b, ix->dirs, ix->jit);
        if (table > 0) orc_gen_table_params(seed, table, G, M, d, ix->Wl, ix->A, ix->b);
        free(D); free(tot); free(mu); free(srt);
    }
    free(tmp); free(s); free(seg); free(nseg); free(order);

    /* b3: hash every point with its leaf's parameters */
    ix->code = (int32_t *)malloc(sizeof(int32_t) * (size_t)(n > 0 ? n : 1) * M);
    ix->key = (u128 *)malloc(sizeof(u128) * (size_t)(n > 0 ? n : 1));
    int bad = 0;
    #pragma omp parallel for schedule(static) reduction(|:bad)
    for (int64_t i = 0; i < n; i++) {
        float t[16];
        int ok = orc_hash(ix, ix->leaf[i], X + i * (int64_t)d, t, ix->code + i * M, NULL);
        if (!ok) bad = 1;
        ix->key[i] = orc_morton(ix->code + i * M, M, ix->B);
    }
    if (bad) { *err = 4; orc_free(ix); return NULL; }

    /* b4: linear array sorted by the bi-level code; buckets = runs */
    orc_entry *ent = (orc_entry *)malloc(sizeof(orc_entry) * (size_t)(n > 0 ? n : 1));
    for (int64_t i = 0; i < n; i++) { ent[i].leaf = ix->leaf[i]; ent[i].key = ix->key[i]; ent[i].id = i; }
    qsort(ent, (size_t)n, sizeof(orc_entry), orc_entry_cmp);
    ix->perm = (int64_t *)malloc(sizeof(int64_t) * (size_t)(n > 0 ? n : 1));
    int64_t nu = 0;
    for (int64_t i = 0; i < n; i++) {
        ix->perm[i] = ent[i].id;
        if (i == 0 || ent[i].leaf != ent[i - 1].leaf || ent[i].key != ent[i - 1].key) nu++;
    }
    ix->nu = nu;
    ix->ukey = (u128 *)malloc(sizeof(u128) * (size_t)(nu > 0 ? nu : 1));
    ix->uleaf = (int32_t *)malloc(sizeof(int32_t) * (size_t)(nu > 0 ? nu : 1));
    ix->uoff = (int64_t *)malloc(sizeof(int64_t) * (size_t)(nu + 1));
    int64_t u = 0;
    for (int64_t i = 0; i < n; i++) {
        if (i == 0 || ent[i].leaf != ent[i - 1].leaf || ent[i].key != ent[i - 1].key) {
            ix->ukey[u] = ent[i].key;
            ix->uleaf[u] = ent[i].leaf;
            ix->uoff[u] = i;
            u++;
        }
    }
    ix->uoff[nu] = n;
    ix->leaf_u = (int64_t *)malloc(sizeof(int64_t) * (size_t)(G + 1));
    for (int g = 0, uu = 0; g <= G; g++) {
        while (uu < nu && ix->uleaf[uu] < g) uu++;
        ix->leaf_u[g] = uu;
    }
    free(ent);
    *err = 0;
    return ix;
}

/* Bucket of (leaf, key): [*s, *e) positions; empty when absent. */
static void orc_lookup(const orc_index *ix, int g, u128 key, int64_t *s, int64_t *e)
{
    *s = *e = 0;
    for (int64_t u = ix->leaf_u[g]; u < ix->leaf_u[g + 1]; u++)
        if (ix->ukey[u] == key) { *s = ix->uoff[u]; *e = ix->uoff[u + 1]; return; }
}

typedef struct { double d2; int64_t id; } orc_nb;

static int orc_nb_cmp(const void *pa, const void *pb)
{
    const orc_nb *a = (const orc_nb *)pa, *b = (const orc_nb *)pb;
    if (a->d2 < b->d2) return -1;
    if (a->d2 > b->d2) return 1;
    return (a->id > b->id) - (a->id < b->id);
}

static double orc_dist2_f64(const float *q, const float *x, int d)
{
    double s = 0.0;
    for (int j = 0; j < d; j++) {
        double e = (double)q[j] - (double)x[j];
        s += e * e;
    }
    return s;
}

static int orc_cmp_i64(const void *a, const void *b)
{
    int64_t x = *(const int64_t *)a, y = *(const int64_t *)b;
    return (x > y) - (x < y);
}

/* Short-list search: exact distance to every candidate,   */
/* keep the k smallest by (d^2, id); pad with (-1, +inf) (R22).             */
static void orc_shortlist(const float *X, int d, const float *q, const int64_t *cand, int64_t nc,
                          int k, int64_t *ids, float *d2)
{
    orc_nb *nb = (orc_nb *)malloc(sizeof(orc_nb) * (size_t)(nc > 0 ? nc : 1));
    for (int64_t i = 0; i < nc; i++) {
        nb[i].d2 = orc_dist2_f64(q, X + cand[i] * (int64_t)d, d);
        nb[i].id = cand[i];
    }
    qsort(nb, (size_t)nc, sizeof(orc_nb), orc_nb_cmp);
    for (int r = 0; r < k; r++) {
        if (r < nc) { ids[r] = nb[r].id; d2[r] = (float)nb[r].d2; }
        else { ids[r] = -1; d2[r] = INFINITY; }
    }
    free(nb);
}

/* Query.  probe: 0 standard, 1 multiprobe (Z^M), 2 lattice (E8 index).
 * hierarchy (Z^M only): Morton-prefix widening (Eq. 7-8)
 * with threshold tau = min_cand, or the lower median of the base counts of
 * this batch when min_cand == 0 (R18).  Returns 0, or 1 on invalid args. */
/* Number of leading bits two B*M-bit Morton keys share ("the number of most
 * significant bits shared"), B*M when equal. */
static int orc_shared_msb(u128 a, u128 b, int BM)
{
    u128 x = a ^ b;
    int len = 0;
    while (x) { len++; x >>= 1; }
    return BM - len;
}

/* hierarchy = 2 (R32): P:132's shared-MSB climb.  curve_perturb (R31): P:132's
 * bit-perturbed repeats of the Morton-curve search (probe = 3). */
static int orc_query_impl(orc_index *ix, const float *Q, int64_t nq, int k, int probe, int T, int hierarchy,
                          int hier_step, int64_t min_cand, int curve_perturb, int msb_min,
                          int64_t *out_ids, float *out_d2, int64_t *out_ncand, int do_shortlist)
{
    const int M = ix->M, d = ix->d, B = ix->B;
    if (k < 1 || T < 1) return 1;
    if (curve_perturb < 0 || curve_perturb > M || (curve_perturb > 0 && probe != 3)) return 1;
    if (hierarchy < 0 || hierarchy > 2 || (hierarchy == 2 && ix->quantizer != 0)) return 1;
    if (msb_min < 0 || msb_min > B * M) return 1;
    if (probe == 0 && T != 1) return 1;
    if (probe == 1 && (ix->quantizer != 0 || M > 10 || T > orc_pow3(M))) return 1;
    if (probe == 2 && (ix->quantizer != 1 || T > 256 || (M == 16 && T > 481))) return 1;
    if (probe == 3 && ix->quantizer != 0) return 1;
    if (probe < 0 || probe > 3) return 1;
    /* hierarchy: Morton prefixes on Z^M (R17), the Eq. 10 code hierarchy on E8 (R27) */
    if (min_cand < 0) return 1;
    int step = hier_step <= 0 ? M : hier_step;
    if (step > M) return 1;
    orc_free_lastq(ix);
    ix->lq_n = nq;
    ix->lq_T = T;
    size_t nqs = (size_t)(nq > 0 ? nq : 1);
    ix->lq_leaf = (int32_t *)calloc(nqs, sizeof(int32_t));
    ix->lq_t = (float *)calloc(nqs * M, sizeof(float));
    ix->lq_code = (int32_t *)calloc(nqs * M, sizeof(int32_t));
    ix->lq_oor = (int32_t *)calloc(nqs, sizeof(int32_t));
    ix->lq_key = (uint64_t *)calloc(nqs * 2, sizeof(uint64_t));
    ix->lq_pkey = (uint64_t *)calloc(nqs * T * 2, sizeof(uint64_t));
    ix->lq_pvalid = (int32_t *)calloc(nqs * T, sizeof(int32_t));
    ix->lq_base = (int64_t *)calloc(nqs, sizeof(int64_t));
    ix->lq_level = (int32_t *)calloc(nqs, sizeof(int32_t));
    ix->lq_coff = (int64_t *)calloc(nqs + 1, sizeof(int64_t));
    int64_t *bs = (int64_t *)malloc(sizeof(int64_t) * nqs * T);   /* probe buckets */
    int64_t *be = (int64_t *)malloc(sizeof(int64_t) * nqs * T);
    int64_t *hs = (int64_t *)calloc(nqs, sizeof(int64_t));        /* hierarchy range */
    int64_t *he = (int64_t *)calloc(nqs, sizeof(int64_t));
    int64_t **hbk = (int64_t **)calloc(nqs, sizeof(int64_t *));   /* E8 hierarchy: node buckets */
    int64_t *nhbk = (int64_t *)calloc(nqs, sizeof(int64_t));
    u128 *hkey = (u128 *)calloc(nqs, sizeof(u128));
    int32_t roots[240 * 8];
    orc_e8_roots(roots);
    int32_t *ring2 = NULL;           /* recursive E8 probing (R26) */
    /* R33 ("If the number of candidates computed is not enough, we
     * recursively probe the adjacent buckets of the 240 probed buckets"): with
     * min_cand = tau > 0 and no hierarchy, the second-ring probes 241..T-1 of
     * the lattice sequence are taken one by one, in sequence order, only while
     * the candidates of the probes before them number fewer than tau; a probe
     * not taken is invalid (key 0, no bucket). */
    const int e8_rec = probe == 2 && hierarchy == 0 && min_cand > 0 && M == 8 && T > 241;
    if (probe == 2 && T > 241 && M == 8) {
        ring2 = (int32_t *)malloc(sizeof(int32_t) * 8 * ORC_E8_S2);
        orc_e8_second_ring(ring2);
    }

    /* a1-a4: route, hash, probe sequence, bucket lookup, base count |A0| */
    #pragma omp parallel for schedule(dynamic, 16)
    for (int64_t q = 0; q < nq; q++) {
        const float *x = Q + q * (int64_t)d;
        int g = orc_route(ix, x);
        float *t = ix->lq_t + q * M;
        int32_t *code = ix->lq_code + q * M;
        int32_t clamped[16];
        int ok = orc_hash(ix, g, x, t, code, clamped);
        /* R30: a non-finite projection (NaN/Inf in the query) has no
         * probe order (its scores are NaN): no probes, no candidates.           */
        int nonfin = 0;
        for (int i = 0; i < M; i++) if (!isfinite(t[i])) nonfin = 1;
        ix->lq_leaf[q] = g;
        ix->lq_oor[q] = nonfin ? 5 : !ok;
        hkey[q] = orc_morton(clamped, M, B);
        u128 hk = ok ? orc_morton(code, M, B) : 0;
        ix->lq_key[2 * q] = (uint64_t)(hk >> 64);
        ix->lq_key[2 * q + 1] = (uint64_t)hk;
        int32_t *deltas = (int32_t *)malloc(sizeof(int32_t) * (size_t)T * 16);
        int32_t ridx[256];
        if (probe == 1 && T > 1 && !nonfin) orc_multiprobe_deltas(t, M, T, deltas, NULL);
        if (probe == 2 && T > 1 && ok && !nonfin) orc_lattice_order_blocks(t, code, M, T, ridx);
        const float lo = -(float)(1 << (B - 1)), hi = (float)((1 << (B - 1)) - 1);
        int64_t base = 0;
        if (probe == 3) {
            /* P:132 Morton-curve neighbours (R25): insertion position of the
             * (clamped) home key among the leaf's sorted bucket keys, then the
             * buckets after / before it alternately: offsets 0, -1, +1, -2, ...
             * With curve_perturb = P > 0 (R31, "perturb some bits of the query
             * Morton code and repeat this process several times"): keys
             * kappa_0 = home key, kappa_r = home key with bit 0 of coordinate c_r
             * flipped (one cell towards +1 if that bit is 0, else towards -1),
             * c_1, c_2, ... = coordinates by ascending (distance to that cell
             * boundary x_i(delta_i) of R11, i); probe j searches around the
             * insertion position of kappa_(j mod (P+1)) with offset number
             * j div (P+1); a bucket already probed is an empty probe. */
            const int R = curve_perturb + 1;
            u128 keys[17];
            keys[0] = hkey[q];
            if (R > 1 && !nonfin) {
                int ord[16];
                float xd[16];
                for (int i = 0; i < M; i++) {
                    const float xm = t[i] - floorf(t[i]);                    /* x_i(-1) */
                    const int up = (((clamped[i] + (1 << (B - 1))) & 1) == 0); /* bit 0 of u_i is 0: +1 */
                    xd[i] = up ? 1.0f - xm : xm;
                    ord[i] = i;
                }
                for (int i = 1; i < M; i++) {          /* insertion sort: ties keep index order */
                    int c = ord[i], j = i - 1;
                    while (j >= 0 && xd[ord[j]] > xd[c]) { ord[j + 1] = ord[j]; j--; }
                    ord[j + 1] = c;
                }
                for (int r = 1; r < R; r++) keys[r] = hkey[q] ^ ((u128)1 << (M - 1 - ord[r - 1]));
            }
            int64_t pr[17];
            for (int r = 0; r < R; r++) {
                pr[r] = ix->leaf_u[g];
                for (int64_t u = ix->leaf_u[g]; u < ix->leaf_u[g + 1]; u++)
                    if (ix->ukey[u] < keys[r]) pr[r] = u + 1;
            }
            int64_t *pb = (int64_t *)malloc(sizeof(int64_t) * (size_t)T);
            for (int p = 0; p < T; p++) {
                const int r = p % R, mo = p / R;
                int64_t off = (mo % 2 == 1) ? -(int64_t)((mo + 1) / 2) : (int64_t)(mo / 2);
                int64_t b = pr[r] + off;
                int valid = !nonfin && b >= ix->leaf_u[g] && b < ix->leaf_u[g + 1];
                for (int pp = 0; pp < p && valid; pp++) if (pb[pp] == b) valid = 0;
                pb[p] = valid ? b : -1;
                u128 pk = valid ? ix->ukey[b] : 0;
                ix->lq_pkey[((size_t)q * T + p) * 2] = (uint64_t)(pk >> 64);
                ix->lq_pkey[((size_t)q * T + p) * 2 + 1] = (uint64_t)pk;
                ix->lq_pvalid[(size_t)q * T + p] = valid;
                bs[(size_t)q * T + p] = valid ? ix->uoff[b] : 0;
                be[(size_t)q * T + p] = valid ? ix->uoff[b + 1] : 0;
                base += be[(size_t)q * T + p] - bs[(size_t)q * T + p];
            }
            free(pb);
        }
        for (int p = 0; p < T && probe != 3; p++) {
            int32_t pc[16];
            int valid = 1;
            if (nonfin) {
                valid = 0;
            } else if (ix->quantizer == 0) {
                /* Z^M: probe code = floor(t) + delta, empty if outside the range (R9) */
                for (int i = 0; i < M; i++) {
                    float f = floorf(t[i]) + (p == 0 ? 0.0f : (float)deltas[(p - 1) * M + i]);
                    if (!(f >= lo && f <= hi)) valid = 0;
                    else pc[i] = (int32_t)f;
                }
            } else if (e8_rec && p > 240 && base >= min_cand) {
                valid = 0;      /* R33: enough candidates, the recursion stops */
            } else {
                /* E8: home c, then c + r for the selected roots */
                valid = ok;
                for (int i = 0; i < M; i++) pc[i] = code[i];
                if (p > 0 && M == 8) {
                    for (int i = 0; i < 8; i++)
                        pc[i] += ridx[p - 1] < 240 ? roots[ridx[p - 1] * 8 + i] : ring2[(ridx[p - 1] - 240) * 8 + i];
                } else if (p > 0) {     /* M = 16: one block moved by one root (R28) */
                    const int blk = ridx[p - 1] / 240, r = ridx[p - 1] % 240;
                    for (int i = 0; i < 8; i++) pc[8 * blk + i] += roots[r * 8 + i];
                }
                if (valid && !orc_code_in_range(pc, M, B)) valid = 0;
            }
            u128 pk = valid ? orc_morton(pc, M, B) : 0;
            ix->lq_pkey[((size_t)q * T + p) * 2] = (uint64_t)(pk >> 64);
            ix->lq_pkey[((size_t)q * T + p) * 2 + 1] = (uint64_t)pk;
            ix->lq_pvalid[(size_t)q * T + p] = valid;
            int64_t s = 0, e = 0;
            if (valid) orc_lookup(ix, g, pk, &s, &e);
            bs[(size_t)q * T + p] = s;
            be[(size_t)q * T + p] = e;
            base += e - s;      /* distinct keys -> disjoint buckets */
        }
        free(deltas);
        ix->lq_base[q] = base;
    }

    /* threshold tau (median of the short-list sizes of the query set) */
    int64_t tau = min_cand;
    if (hierarchy == 1 && min_cand == 0 && nq > 0) {
        int64_t *c = (int64_t *)malloc(sizeof(int64_t) * nqs);
        memcpy(c, ix->lq_base, sizeof(int64_t) * nqs);
        qsort(c, (size_t)nq, sizeof(int64_t), orc_cmp_i64);
        tau = c[(nq - 1) / 2];
        free(c);
    }
    ix->lq_tau = hierarchy == 1 ? tau : 0;

    /* E8 hierarchy (R27): a node at level j = the leaf's buckets whose
     * level-j code equals the query's; matches are closed upwards (the level-j+1
     * code is a function of the level-j code).  The traversal descends from the
     * root (level m_g: the first level where all the leaf's buckets share one
     * code, <= ORC_E8_LEVELS) to the deepest node matching the query,
     * and P:249 widens from there until the node holds >= tau points: the first
     * level j <= m_g with a match and |node| >= tau; otherwise the whole leaf. */
    if (hierarchy == 1 && ix->quantizer == 1) {
        #pragma omp parallel for schedule(dynamic, 4)
        for (int64_t q = 0; q < nq; q++) {
            if (ix->lq_base[q] >= tau || (ix->lq_oor[q] & 4)) continue;
            int g = ix->lq_leaf[q];
            int64_t u0 = ix->leaf_u[g], nb = ix->leaf_u[g + 1] - u0;
            int32_t *cur = (int32_t *)malloc(sizeof(int32_t) * M * (size_t)(nb > 0 ? nb : 1));
            int32_t cq[16], tmp[16];
            const size_t cb = sizeof(int32_t) * (size_t)M;
            memcpy(cq, ix->lq_code + q * M, cb);
            for (int64_t b = 0; b < nb; b++)
                memcpy(cur + M * b, ix->code + M * ix->perm[ix->uoff[u0 + b]], cb);
            int level = ORC_E8_LEVELS + 1;      /* whole leaf */
            for (int jl = 0; jl <= ORC_E8_LEVELS && nb > 0; jl++) {
                int64_t rows = 0, match = 0;
                int same = 1;
                for (int64_t b = 0; b < nb; b++) {
                    if (memcmp(cur + M * b, cq, cb) == 0) {
                        match++;
                        rows += ix->uoff[u0 + b + 1] - ix->uoff[u0 + b];
                    }
                    if (memcmp(cur + M * b, cur, cb) != 0) same = 0;
                }
                if (match && rows >= tau) { level = jl; break; }
                if (same) break;                 /* root reached without a large enough match */
                for (int64_t b = 0; b < nb; b++) {
                    for (int k2 = 0; k2 < M / 8; k2++) orc_e8_parent(cur + M * b + 8 * k2, tmp + 8 * k2);
                    memcpy(cur + M * b, tmp, cb);
                }
                for (int k2 = 0; k2 < M / 8; k2++) orc_e8_parent(cq + 8 * k2, tmp + 8 * k2);
                memcpy(cq, tmp, cb);
            }
            /* node buckets */
            int64_t *lst = (int64_t *)malloc(sizeof(int64_t) * (size_t)(nb > 0 ? nb : 1));
            int64_t m = 0;
            if (level > ORC_E8_LEVELS) {
                for (int64_t b = 0; b < nb; b++) lst[m++] = u0 + b;
            } else {
                /* recompute the level-`level` codes (cur holds them after the loop broke there) */
                for (int64_t b = 0; b < nb; b++)
                    if (memcmp(cur + M * b, cq, cb) == 0) lst[m++] = u0 + b;
            }
            hbk[q] = lst;
            nhbk[q] = m;
            ix->lq_level[q] = level;
            free(cur);
        }
    }

    /* hierarchy: widen along Morton prefixes until |R| >= tau (Eq. 8) */
    if (hierarchy == 1 && ix->quantizer == 0) {
        const int BM = B * M;
        #pragma omp parallel for schedule(dynamic, 16)
        for (int64_t q = 0; q < nq; q++) {
            if (ix->lq_base[q] >= tau || (ix->lq_oor[q] & 4)) continue;
            int g = ix->lq_leaf[q];
            for (int l = 1;; l++) {
                int cb = l * step < BM ? l * step : BM;
                u128 mask = cb >= 128 ? ~(u128)0 : (((u128)1 << cb) - 1);
                u128 lo = hkey[q] & ~mask, hi = lo | mask;
                int64_t s = -1, e = -1;
                for (int64_t u = ix->leaf_u[g]; u < ix->leaf_u[g + 1]; u++) {
                    if (ix->ukey[u] >= lo && ix->ukey[u] <= hi) {
                        if (s < 0) s = ix->uoff[u];
                        e = ix->uoff[u + 1];
                    }
                }
                if (s < 0) { s = 0; e = 0; }
                if (e - s >= tau || cb == BM) {
                    hs[q] = s; he[q] = e; ix->lq_level[q] = cb;
                    break;
                }
            }
        }
    }

    /* P:132 shared-MSB climb (R32, hierarchy = 2): s* = the larger number of
     * most significant bits the (clamped) home key shares with the keys just
     * before and after its insertion position in the leaf's sorted keys; when
     * s* is small (< msb_min, default B*M: the home bucket is empty) the query
     * goes up to the level of s* shared bits and uses that larger bucket, the
     * leaf's buckets whose keys share those s* bits with it: A = A0 u R. */
    if (hierarchy == 2) {
        const int BM = B * M;
        const int sig = msb_min > 0 ? msb_min : BM;
        #pragma omp parallel for schedule(dynamic, 16)
        for (int64_t q = 0; q < nq; q++) {
            if (ix->lq_oor[q] & 4) continue;
            int g = ix->lq_leaf[q];
            int64_t ul = ix->leaf_u[g], uh = ix->leaf_u[g + 1];
            if (uh <= ul) continue;
            int64_t p0 = ul;
            for (int64_t u = ul; u < uh; u++) if (ix->ukey[u] < hkey[q]) p0 = u + 1;
            int sstar = 0;
            if (p0 > ul) { int c = orc_shared_msb(hkey[q], ix->ukey[p0 - 1], BM); if (c > sstar) sstar = c; }
            if (p0 < uh) { int c = orc_shared_msb(hkey[q], ix->ukey[p0], BM); if (c > sstar) sstar = c; }
            if (sstar >= sig) continue;
            int cb = BM - sstar;
            u128 mask = cb >= 128 ? ~(u128)0 : (((u128)1 << cb) - 1);
            u128 lo = hkey[q] & ~mask, hi = lo | mask;
            int64_t s = -1, e = -1;
            for (int64_t u = ul; u < uh; u++) {
                if (ix->ukey[u] >= lo && ix->ukey[u] <= hi) {
                    if (s < 0) s = ix->uoff[u];
                    e = ix->uoff[u + 1];
                }
            }
            if (s < 0) { s = 0; e = 0; }
            hs[q] = s; he[q] = e; ix->lq_level[q] = cb;
        }
    }

    /* C7: A(q) = distinct points of the probed buckets / range of the leaf */
    int64_t **cand = (int64_t **)calloc(nqs, sizeof(int64_t *));
    int64_t *ncand = (int64_t *)calloc(nqs, sizeof(int64_t));
    #pragma omp parallel for schedule(dynamic, 16)
    for (int64_t q = 0; q < nq; q++) {
        int64_t cap = ix->lq_base[q] + (he[q] - hs[q]);
        for (int64_t b = 0; b < nhbk[q]; b++) cap += ix->uoff[hbk[q][b] + 1] - ix->uoff[hbk[q][b]];
        int64_t *pos = (int64_t *)malloc(sizeof(int64_t) * (size_t)(cap > 0 ? cap : 1));
        int64_t np = 0;
        for (int p = 0; p < T; p++)
            for (int64_t i = bs[(size_t)q * T + p]; i < be[(size_t)q * T + p]; i++) pos[np++] = i;
        for (int64_t i = hs[q]; i < he[q]; i++) pos[np++] = i;
        for (int64_t b = 0; b < nhbk[q]; b++)
            for (int64_t i = ix->uoff[hbk[q][b]]; i < ix->uoff[hbk[q][b] + 1]; i++) pos[np++] = i;
        free(hbk[q]);
        qsort(pos, (size_t)np, sizeof(int64_t), orc_cmp_i64);
        int64_t m = 0;
        for (int64_t i = 0; i < np; i++) if (m == 0 || pos[i] != pos[m - 1]) pos[m++] = pos[i];
        for (int64_t i = 0; i < m; i++) pos[i] = ix->perm[pos[i]];
        qsort(pos, (size_t)m, sizeof(int64_t), orc_cmp_i64);
        cand[q] = pos;
        ncand[q] = m;
        if (out_ncand) out_ncand[q] = m;
        /* a5: short-list search */
        if (do_shortlist)
            orc_shortlist(ix->X, d, Q + q * (int64_t)d, pos, m, k, out_ids + q * (int64_t)k,
                          out_d2 + q * (int64_t)k);
    }
    ix->lq_coff[0] = 0;
    for (int64_t q = 0; q < nq; q++) ix->lq_coff[q + 1] = ix->lq_coff[q] + ncand[q];
    ix->lq_cand = (int64_t *)malloc(sizeof(int64_t) * (size_t)(ix->lq_coff[nq] > 0 ? ix->lq_coff[nq] : 1));
    for (int64_t q = 0; q < nq; q++) {
        memcpy(ix->lq_cand + ix->lq_coff[q], cand[q], sizeof(int64_t) * (size_t)ncand[q]);
        free(cand[q]);
    }
    free(cand); free(ncand); free(bs); free(be); free(hs); free(he); free(hkey); free(hbk); free(nhbk); free(ring2);
    return 0;
}

int orc_query(orc_index *ix, const float *Q, int64_t nq, int k, int probe, int T, int hierarchy,
              int hier_step, int64_t min_cand, int64_t *out_ids, float *out_d2, int64_t *out_ncand)
{
    return orc_query_impl(ix, Q, nq, k, probe, T, hierarchy, hier_step, min_cand, 0, 0, out_ids, out_d2,
                          out_ncand, 1);
}

/* orc_query with P:132's remaining options: curve_perturb (R31) and the shared-MSB
 * climb threshold msb_min (R32, hierarchy = 2; 0 = B*M). */
int orc_query_ex(orc_index *ix, const float *Q, int64_t nq, int k, int probe, int T, int hierarchy,
                 int hier_step, int64_t min_cand, int curve_perturb, int msb_min, int64_t *out_ids,
                 float *out_d2, int64_t *out_ncand)
{
    return orc_query_impl(ix, Q, nq, k, probe, T, hierarchy, hier_step, min_cand, curve_perturb, msb_min,
                          out_ids, out_d2, out_ncand, 1);
}

/* L > 1 tables: "each of them is constructed independently with
 * different dim-M hash functions"; the candidate set of a query is the union
 * of the points of its probed buckets over the L tables, deduplicated (R24:
 * every table probes T buckets the same way; the Morton hierarchy is not
 * combined with L > 1).  tabs[l] is the index built with table = l (same
 * data, tree and seed).  Short-list as for one table.  Returns 0, or 1 on
 * invalid arguments. */
int orc_query_union(orc_index **tabs, int L, const float *Q, int64_t nq, int k, int probe, int T,
                    int64_t *out_ids, float *out_d2, int64_t *out_ncand)
{
    if (L < 1) return 1;
    for (int l = 0; l < L; l++)
        if (orc_query_impl(tabs[l], Q, nq, k, probe, T, 0, 0, 0, 0, 0, out_ids, out_d2, NULL, 0)) return 1;
    const int d = tabs[0]->d;
    #pragma omp parallel for schedule(dynamic, 16)
    for (int64_t q = 0; q < nq; q++) {
        int64_t cap = 0;
        for (int l = 0; l < L; l++) cap += tabs[l]->lq_coff[q + 1] - tabs[l]->lq_coff[q];
        int64_t *ids = (int64_t *)malloc(sizeof(int64_t) * (size_t)(cap > 0 ? cap : 1));
        int64_t m = 0;
        for (int l = 0; l < L; l++)
            for (int64_t i = tabs[l]->lq_coff[q]; i < tabs[l]->lq_coff[q + 1]; i++) ids[m++] = tabs[l]->lq_cand[i];
        qsort(ids, (size_t)m, sizeof(int64_t), orc_cmp_i64);
        int64_t u = 0;
        for (int64_t i = 0; i < m; i++) if (u == 0 || ids[i] != ids[u - 1]) ids[u++] = ids[i];
        if (out_ncand) out_ncand[q] = u;
        orc_shortlist(tabs[0]->X, d, Q + q * (int64_t)d, ids, u, k, out_ids + q * (int64_t)k,
                      out_d2 + q * (int64_t)k);
        free(ids);
    }
    return 0;
}

/* Exact k-NN by brute force in fp64 (P:33 definition of I(v) / N(v)). */
void orc_bruteforce(const float *X, int64_t n, int d, const float *Q, int64_t nq, int k,
                    int64_t *out_ids, float *out_d2)
{
    #pragma omp parallel for schedule(dynamic, 1)
    for (int64_t q = 0; q < nq; q++) {
        const float *x = Q + q * (int64_t)d;
        orc_nb *best = (orc_nb *)malloc(sizeof(orc_nb) * (size_t)k);
        int nb = 0;
        for (int64_t i = 0; i < n; i++) {
            double s = orc_dist2_f64(x, X + i * (int64_t)d, d);
            if (nb == k && !(s < best[k - 1].d2 || (s == best[k - 1].d2 && i < best[k - 1].id))) continue;
            int p = nb < k ? nb : k - 1;
            while (p > 0 && (best[p - 1].d2 > s || (best[p - 1].d2 == s && best[p - 1].id > i))) {
                best[p] = best[p - 1];
                p--;
            }
            best[p].d2 = s;
            best[p].id = i;
            if (nb < k) nb++;
        }
        for (int r = 0; r < k; r++) {
            if (r < nb) { out_ids[q * k + r] = best[r].id; out_d2[q * k + r] = (float)best[r].d2; }
            else { out_ids[q * k + r] = -1; out_d2[q * k + r] = INFINITY; }
        }
        free(best);
    }
}

/* ------------------------------------------------------------------------ */
/* Accessors for tests (copy-out of build artefacts and last-query stages). */
/* ------------------------------------------------------------------------ */
void orc_info(const orc_index *ix, int64_t *out /* [8] */)
{
    out[0] = ix->n; out[1] = ix->d; out[2] = ix->G; out[3] = ix->M;
    out[4] = ix->B; out[5] = ix->nu; out[6] = ix->lq_n; out[7] = ix->lq_tau;
}

int64_t orc_last_ncand_total(const orc_index *ix) { return ix->lq_n ? ix->lq_coff[ix->lq_n] : 0; }

/* what: 0 A, 1 b, 2 dirs, 3 theta, 4 ntype, 5 mu, 6 leaf, 7 code, 8 key(hi,lo),
 * 9 perm, 10 ukey(hi,lo), 11 uleaf, 12 uoff, 13 leaf_u, 14 W, 15 diam2, 16 da2,
 * 17 jit.   Query stages: 20 leaf, 21 t, 22 code, 23 oor, 24 key, 25 probe keys,
 * 26 probe valid, 27 base count, 28 level, 29 cand offsets, 30 cand ids. */
int orc_get(const orc_index *ix, int what, void *dst)
{
    const int64_t n = ix->n, G = ix->G, M = ix->M, d = ix->d, nn = G > 1 ? G - 1 : 0;
    const int64_t nq = ix->lq_n;
    switch (what) {
    case 0: memcpy(dst, ix->A, sizeof(float) * G * M * d); return 0;
    case 1: memcpy(dst, ix->b, sizeof(float) * G * M); return 0;
    case 2: memcpy(dst, ix->dirs, sizeof(float) * nn * d); return 0;
    case 3: memcpy(dst, ix->theta, sizeof(float) * nn); return 0;
    case 4: memcpy(dst, ix->ntype, sizeof(int32_t) * nn); return 0;
    case 5: memcpy(dst, ix->mu, sizeof(float) * nn * d); return 0;
    case 6: memcpy(dst, ix->leaf, sizeof(int32_t) * n); return 0;
    case 7: memcpy(dst, ix->code, sizeof(int32_t) * n * M); return 0;
    case 8: {
        uint64_t *o = (uint64_t *)dst;
        for (int64_t i = 0; i < n; i++) { o[2 * i] = (uint64_t)(ix->key[i] >> 64); o[2 * i + 1] = (uint64_t)ix->key[i]; }
        return 0;
    }
    case 9: memcpy(dst, ix->perm, sizeof(int64_t) * n); return 0;
    case 10: {
        uint64_t *o = (uint64_t *)dst;
        for (int64_t i = 0; i < ix->nu; i++) { o[2 * i] = (uint64_t)(ix->ukey[i] >> 64); o[2 * i + 1] = (uint64_t)ix->ukey[i]; }
        return 0;
    }
    case 11: memcpy(dst, ix->uleaf, sizeof(int32_t) * ix->nu); return 0;
    case 12: memcpy(dst, ix->uoff, sizeof(int64_t) * (ix->nu + 1)); return 0;
    case 13: memcpy(dst, ix->leaf_u, sizeof(int64_t) * (G + 1)); return 0;
    case 14: memcpy(dst, ix->Wl, sizeof(float) * G); return 0;
    case 15: memcpy(dst, ix->diam2, sizeof(double) * nn); return 0;
    case 16: memcpy(dst, ix->da2, sizeof(double) * nn); return 0;
    case 17: memcpy(dst, ix->jit, sizeof(double) * nn); return 0;
    case 20: memcpy(dst, ix->lq_leaf, sizeof(int32_t) * nq); return 0;
    case 21: memcpy(dst, ix->lq_t, sizeof(float) * nq * M); return 0;
    case 22: memcpy(dst, ix->lq_code, sizeof(int32_t) * nq * M); return 0;
    case 23: memcpy(dst, ix->lq_oor, sizeof(int32_t) * nq); return 0;
    case 24: memcpy(dst, ix->lq_key, sizeof(uint64_t) * nq * 2); return 0;
    case 25: memcpy(dst, ix->lq_pkey, sizeof(uint64_t) * nq * ix->lq_T * 2); return 0;
    case 26: memcpy(dst, ix->lq_pvalid, sizeof(int32_t) * nq * ix->lq_T); return 0;
    case 27: memcpy(dst, ix->lq_base, sizeof(int64_t) * nq); return 0;
    case 28: memcpy(dst, ix->lq_level, sizeof(int32_t) * nq); return 0;
    case 29: memcpy(dst, ix->lq_coff, sizeof(int64_t) * (nq + 1)); return 0;
    case 30: memcpy(dst, ix->lq_cand, sizeof(int64_t) * ix->lq_coff[nq]); return 0;
    default: return 1;
    }
}

int orc_num_threads(void)
{
#ifdef _OPENMP
    return omp_get_max_threads();
#else
    return 1;
#endif
}

void orc_set_num_threads(int n)
{
#ifdef _OPENMP
    if (n > 0) omp_set_num_threads(n);
#else
    (void)n;
#endif
}
