// params.cpp -- b1: seeded LSH parameters and RP directions (host).
//
// Reading R2: counter-based SplitMix64, Box-Muller (cosine
// branch) in fp64, streams kind<<24 | table<<16 | leaf_or_node.  P:43 draws
// a_i ~ N(0,1) and b_i ~ U[0,W); P:98 a random unit direction per node.
// Compiled with -ffp-contract=off: every a*b+c below is two roundings unless
// written as std::fma.
#include <cmath>
#include <cstdint>
#include <vector>

namespace blsh {

namespace {
constexpr uint64_t kGamma = 0x9E3779B97F4A7C15ull;

inline uint64_t splitmix(uint64_t z) {
    z ^= z >> 30;
    z *= 0xBF58476D1CE4E5B9ull;
    z ^= z >> 27;
    z *= 0x94D049BB133111EBull;
    z ^= z >> 31;
    return z;
}
inline uint64_t counter_u64(uint64_t seed, uint64_t stream, uint64_t i) {
    return splitmix(seed + kGamma * ((stream << 32) + i + 1ull));
}
inline double counter_uniform(uint64_t seed, uint64_t stream, uint64_t i) {
    return (double)(counter_u64(seed, stream, i) >> 11) * 0x1.0p-53;
}
inline double counter_normal(uint64_t seed, uint64_t stream, uint64_t i) {
    const double u1 = counter_uniform(seed, stream, 2 * i);
    const double u2 = counter_uniform(seed, stream, 2 * i + 1);
    return std::sqrt(-2.0 * std::log(1.0 - u1)) * std::cos(2.0 * 3.141592653589793 * u2);
}
inline uint64_t stream_id(uint64_t kind, uint64_t table, uint64_t idx) {
    return (kind << 24) + (table << 16) + idx;
}
}  // namespace

// L tables "constructed independently with different dim-M hash
// functions": table l draws (a, b) from streams (1, l, g) and (2, l, g).
void gen_table_params(uint64_t seed, int table, int G, int M, int d, const float* Wleaf, float* A, float* b) {
    for (int g = 0; g < G; ++g) {
        const uint64_t sa = stream_id(1, (uint64_t)table, (uint64_t)g), sb = stream_id(2, (uint64_t)table, (uint64_t)g);
        for (int i = 0; i < M; ++i)
            for (int j = 0; j < d; ++j)
                A[((size_t)g * M + i) * d + j] = (float)counter_normal(seed, sa, (uint64_t)i * d + j);
        for (int i = 0; i < M; ++i) {
            const float W = Wleaf[g];
            float v = (float)((double)W * counter_uniform(seed, sb, (uint64_t)i));
            if (v >= W) v = std::nextafter(W, 0.0f);
            b[(size_t)g * M + i] = v;
        }
    }
}

void gen_params(uint64_t seed, int G, int M, int d, const float* Wleaf, float* A, float* b,
                float* dirs, double* jit) {
    gen_table_params(seed, 0, G, M, d, Wleaf, A, b);
    std::vector<double> gv((size_t)d);
    for (int v = 0; v + 1 < G; ++v) {
        const uint64_t sd = stream_id(3, 0, (uint64_t)v);
        double ss = 0.0;
        for (int j = 0; j < d; ++j) {
            gv[j] = counter_normal(seed, sd, (uint64_t)j);
            ss = std::fma(gv[j], gv[j], ss);
        }
        const double nrm = std::sqrt(ss);
        for (int j = 0; j < d; ++j) dirs[(size_t)v * d + j] = (float)(gv[j] / nrm);
        jit[v] = counter_uniform(seed, stream_id(4, 0, (uint64_t)v), 0);
    }
}

}  // namespace blsh
