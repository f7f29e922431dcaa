// rptree.cu -- b2: level I of Bi-level LSH, the RP-tree.
//
// Built level by level.  Members of every node are kept contiguous in `order`
// in ascending id (a stable partition per level), so every per-node quantity
// is a segmented pass over HBM:
//   * mean rule: mean mu, Delta_A^2 = 2 sum dist2c(x, mu) / |S| with the
//     ordered fp64 reductions of R7, the approximate diameter of R6
//     (m = ek_iters passes), the test Delta^2 <= c Delta_A^2;
//   * split value s(x) = dot(dir, x) (hyperplane) or dist2c(x, mu) (sphere);
//   * exact lower median by a 4-pass segmented radix select (R5);
//   * stable partition (x left iff s(x) <= theta).
// All per-row chains are the canonical fp32 chains of R1, computed by
// `k_rowchain` on 256-row tiles staged through shared memory 32 columns at a
// time (coalesced 128-byte row segments; conflict-free reads with a 33-float
// row pitch).
#include <algorithm>
#include <cmath>

#include "internal.cuh"

namespace blsh {

namespace {

constexpr int kTR = 256;       // rows per tile (one thread per row)
constexpr int kDC = 32;        // columns per shared-memory stage
constexpr int kChunk = 4096;   // R7 reduction chunk

struct Tile {
    int32_t node;    // heap index
    int32_t len;
    int64_t start;   // position in order
};
struct Chunk {
    int32_t node;
    int32_t len;
    int64_t start;
};

enum { RC_DOT = 0, RC_DIST = 1, RC_SPLIT = 2 };

// Canonical chain per row of a tile against one vector per node.
//   RC_DOT:   s = fmaf chain of vec[j] * x[j]            (vec = vbase + node*ds)
//   RC_DIST:  s = fmaf chain of (x[j]-vec[j])^2           (vec = vbase + vrow[node]*ds, or + node*ds)
//   RC_SPLIT: node type 0 -> RC_DOT with dirs, type 1 -> RC_DIST with mu
template <int MODE>
__global__ void __launch_bounds__(kTR) k_rowchain(const float* __restrict__ Xs, int ds, int d,
                                                  const uint32_t* __restrict__ order,
                                                  const Tile* __restrict__ tiles,
                                                  const float* __restrict__ vbase,
                                                  const uint32_t* __restrict__ vrow,
                                                  const int32_t* __restrict__ ntype,
                                                  const float* __restrict__ vbase2,
                                                  float* __restrict__ out) {
    __shared__ float xs[kTR][kDC + 1];
    __shared__ float vs[kDC];
    __shared__ uint32_t rid[kTR];
    const Tile t = tiles[blockIdx.x];
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const int r = threadIdx.x;
    if (r < t.len) rid[r] = order[t.start + r];
    bool dist;
    const float* vec;
    if (MODE == RC_SPLIT) {
        dist = ntype[t.node] != 0;
        vec = (dist ? vbase2 : vbase) + (size_t)t.node * ds;
    } else {
        dist = MODE == RC_DIST;
        vec = vbase + (size_t)(vrow ? vrow[t.node] : (uint32_t)t.node) * ds;
    }
    __syncthreads();
    float s = 0.0f;
    for (int dc = 0; dc < d; dc += kDC) {
        const int w = min(kDC, d - dc);
#pragma unroll 4
        for (int rr = warp; rr < t.len; rr += kTR / 32)
            if (lane < w) xs[rr][lane] = Xs[(size_t)rid[rr] * ds + dc + lane];
        if (threadIdx.x < w) vs[threadIdx.x] = vec[dc + threadIdx.x];
        __syncthreads();
        if (r < t.len) {
            if (dist) {
                for (int jj = 0; jj < w; ++jj) {
                    const float e = __fsub_rn(xs[r][jj], vs[jj]);
                    s = __fmaf_rn(e, e, s);
                }
            } else {
                for (int jj = 0; jj < w; ++jj) s = __fmaf_rn(vs[jj], xs[r][jj], s);
            }
        }
        __syncthreads();
    }
    if (r < t.len) out[t.start + r] = s;
}

// Column sums per chunk (R7): part[c][j] = sequential fp64 sum over the chunk.
__global__ void k_colsum(const float* __restrict__ Xs, int ds, int d, const uint32_t* __restrict__ order,
                         const Chunk* __restrict__ chunks, double* __restrict__ part) {
    const Chunk c = chunks[blockIdx.x];
    const int j = blockIdx.y * blockDim.x + threadIdx.x;
    if (j >= d) return;
    double p = 0.0;
    int i = 0;
    for (; i + 8 <= c.len; i += 8) {
        uint32_t id[8];
        float v[8];
#pragma unroll
        for (int u = 0; u < 8; ++u) id[u] = order[c.start + i + u];
#pragma unroll
        for (int u = 0; u < 8; ++u) v[u] = Xs[(size_t)id[u] * ds + j];
#pragma unroll
        for (int u = 0; u < 8; ++u) p = __dadd_rn(p, (double)v[u]);
    }
    for (; i < c.len; ++i) p = __dadd_rn(p, (double)Xs[(size_t)order[c.start + i] * ds + j]);
    part[(size_t)blockIdx.x * d + j] = p;
}

// mu[v][j] = fp32( (sum over the node's chunks, in order) / |S| ).
__global__ void k_mean_final(const double* __restrict__ part, const int64_t* __restrict__ chunk_off,
                             const int64_t* __restrict__ nsz, int node0, int d, int ds,
                             float* __restrict__ mu) {
    const int k = blockIdx.x;
    const int j = blockIdx.y * blockDim.x + threadIdx.x;
    if (j >= d) return;
    double tot = 0.0;
    for (int64_t c = chunk_off[k]; c < chunk_off[k + 1]; ++c) tot = __dadd_rn(tot, part[(size_t)c * d + j]);
    const int64_t n = nsz[k];
    mu[(size_t)(node0 + k) * ds + j] = n > 0 ? __double2float_rn(__ddiv_rn(tot, (double)n)) : 0.0f;
}

// Sequential fp64 sum of vals over each chunk.
__global__ void k_chunksum(const float* __restrict__ vals, const Chunk* __restrict__ chunks, int nchunks,
                           double* __restrict__ out) {
    const int c = blockIdx.x * blockDim.x + threadIdx.x;
    if (c >= nchunks) return;
    const Chunk ch = chunks[c];
    double p = 0.0;
    for (int i = 0; i < ch.len; ++i) p = __dadd_rn(p, (double)vals[ch.start + i]);
    out[c] = p;
}

__global__ void k_da_final(const double* __restrict__ csum, const int64_t* __restrict__ chunk_off,
                           const int64_t* __restrict__ nsz, int nodes, double* __restrict__ da2) {
    const int k = blockIdx.x * blockDim.x + threadIdx.x;
    if (k >= nodes) return;
    double tot = 0.0;
    for (int64_t c = chunk_off[k]; c < chunk_off[k + 1]; ++c) tot = __dadd_rn(tot, csum[c]);
    const int64_t n = nsz[k];
    da2[k] = n > 0 ? __ddiv_rn(__dmul_rn(2.0, tot), (double)n) : 0.0;
}

// Per tile: (optionally acc += vals) and argmax of the metric (ties -> lowest position).
__global__ void __launch_bounds__(kTR) k_argmax_tiles(const float* __restrict__ vals, double* __restrict__ acc,
                                                      int accumulate, const Tile* __restrict__ tiles,
                                                      double* __restrict__ best_v, int64_t* __restrict__ best_p) {
    __shared__ double sv[kTR / 32];
    __shared__ int64_t sp[kTR / 32];
    const Tile t = tiles[blockIdx.x];
    const int r = threadIdx.x;
    double v = -1.0;
    int64_t p = INT64_MAX;
    if (r < t.len) {
        const int64_t pos = t.start + r;
        if (accumulate) {
            v = __dadd_rn(acc[pos], (double)vals[pos]);
            acc[pos] = v;
        } else {
            v = (double)vals[pos];
        }
        p = pos;
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        const double ov = __shfl_xor_sync(BLSH_FULL, v, o);
        const int64_t op = __shfl_xor_sync(BLSH_FULL, p, o);
        if (ov > v || (ov == v && op < p)) { v = ov; p = op; }
    }
    if ((r & 31) == 0) { sv[r >> 5] = v; sp[r >> 5] = p; }
    __syncthreads();
    if (r == 0) {
        for (int w = 1; w < kTR / 32; ++w)
            if (sv[w] > v || (sv[w] == v && sp[w] < p)) { v = sv[w]; p = sp[w]; }
        best_v[blockIdx.x] = v;
        best_p[blockIdx.x] = p;
    }
}

// Per node: best over the node's tiles -> selected point id; writes vrow[node].
__global__ void k_argmax_nodes(const double* __restrict__ best_v, const int64_t* __restrict__ best_p,
                               const int64_t* __restrict__ tile_off, const int32_t* __restrict__ tile_node,
                               int ntiles_nodes, const uint32_t* __restrict__ order,
                               uint32_t* __restrict__ vrow, uint32_t* __restrict__ sel, int it, int m) {
    const int i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= ntiles_nodes) return;
    double v = -1.0;
    int64_t p = INT64_MAX;
    for (int64_t t = tile_off[i]; t < tile_off[i + 1]; ++t)
        if (best_v[t] > v || (best_v[t] == v && best_p[t] < p)) { v = best_v[t]; p = best_p[t]; }
    if (p == INT64_MAX) return;
    const int node = tile_node[i];
    const uint32_t id = order[p];
    vrow[node] = id;
    sel[(size_t)node * m + it] = id;
}

// Max canonical dist2 over pairs of the m selected points of each node (R6).
__global__ void k_pairmax(const float* __restrict__ Xs, int ds, int d, const uint32_t* __restrict__ sel,
                          const int32_t* __restrict__ mnode, const int32_t* __restrict__ node_ids, int m,
                          double* __restrict__ diam2) {
    __shared__ float sm[32];
    const int i = blockIdx.x;
    const int node = node_ids[i];
    const int mv = mnode[i];
    float best = 0.0f;
    const int npairs = mv * (mv - 1) / 2;
    for (int pidx = threadIdx.x; pidx < npairs; pidx += blockDim.x) {
        int a = 0, rem = pidx;
        while (rem >= mv - 1 - a) { rem -= mv - 1 - a; ++a; }
        const int b = a + 1 + rem;
        const float* x = Xs + (size_t)sel[(size_t)node * m + a] * ds;
        const float* y = Xs + (size_t)sel[(size_t)node * m + b] * ds;
        float s = 0.0f;
        for (int j = 0; j < d; ++j) {
            const float e = __fsub_rn(x[j], y[j]);
            s = __fmaf_rn(e, e, s);
        }
        best = fmaxf(best, s);
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) best = fmaxf(best, __shfl_xor_sync(BLSH_FULL, best, o));
    if ((threadIdx.x & 31) == 0) sm[threadIdx.x >> 5] = best;
    __syncthreads();
    if (threadIdx.x == 0) {
        for (int w = 1; w < (int)(blockDim.x >> 5); ++w) best = fmaxf(best, sm[w]);
        diam2[i] = (double)best;
    }
}

// Segmented radix-select histogram (one 8-bit digit of fkey(s)).
__global__ void __launch_bounds__(kTR) k_sel_hist(const float* __restrict__ vals, const Tile* __restrict__ tiles,
                                                  int node0, const uint32_t* __restrict__ prefix, int shift,
                                                  uint32_t* __restrict__ hist) {
    __shared__ uint32_t h[256];
    h[threadIdx.x] = 0;
    __syncthreads();
    const Tile t = tiles[blockIdx.x];
    const int k = t.node - node0;
    if ((int)threadIdx.x < t.len) {
        const uint32_t key = fkey(vals[t.start + threadIdx.x]);
        const bool match = shift == 24 ? true : ((key ^ prefix[k]) >> (shift + 8)) == 0;
        if (match) atomicAdd(&h[(key >> shift) & 255u], 1u);
    }
    __syncthreads();
    if (h[threadIdx.x]) atomicAdd(&hist[(size_t)k * 256 + threadIdx.x], h[threadIdx.x]);
}

__global__ void __launch_bounds__(256) k_sel_pick(uint32_t* __restrict__ hist, uint32_t* __restrict__ prefix,
                                                  int64_t* __restrict__ rank, const int64_t* __restrict__ nsz,
                                                  int shift) {
    __shared__ uint32_t h[256];
    const int k = blockIdx.x;
    h[threadIdx.x] = hist[(size_t)k * 256 + threadIdx.x];
    hist[(size_t)k * 256 + threadIdx.x] = 0;
    __syncthreads();
    if (threadIdx.x == 0 && nsz[k] > 0) {
        int64_t r = rank[k], cum = 0;
        for (int dg = 0; dg < 256; ++dg) {
            if (r < cum + (int64_t)h[dg]) {
                prefix[k] |= (uint32_t)dg << shift;
                rank[k] = r - cum;
                break;
            }
            cum += h[dg];
        }
    }
}

__global__ void k_theta(const uint32_t* __restrict__ prefix, const int64_t* __restrict__ nsz, int nodes,
                        float* __restrict__ theta_level) {
    const int k = blockIdx.x * blockDim.x + threadIdx.x;
    if (k >= nodes) return;
    theta_level[k] = nsz[k] > 0 ? fkey_inv(prefix[k]) : 0.0f;
}

__global__ void __launch_bounds__(kTR) k_left_flags(const float* __restrict__ vals, const Tile* __restrict__ tiles,
                                                    const float* __restrict__ theta, uint8_t* __restrict__ left) {
    const Tile t = tiles[blockIdx.x];
    if ((int)threadIdx.x < t.len) {
        const int64_t pos = t.start + threadIdx.x;
        left[pos] = vals[pos] <= theta[t.node] ? 1 : 0;
    }
}

__global__ void __launch_bounds__(kTR) k_partition(const uint32_t* __restrict__ order, const uint8_t* __restrict__ left,
                                                   const int64_t* __restrict__ L, const Tile* __restrict__ tiles,
                                                   const int64_t* __restrict__ seg, int node0,
                                                   uint32_t* __restrict__ order_new) {
    const Tile t = tiles[blockIdx.x];
    if ((int)threadIdx.x >= t.len) return;
    const int k = t.node - node0;
    const int64_t a = seg[k], e = seg[k + 1];
    const int64_t pos = t.start + threadIdx.x;
    const int64_t la = L[a];
    const int64_t nl = L[e] - la;
    const int64_t rl = L[pos] - la;
    const int64_t dst = left[pos] ? a + rl : a + nl + (pos - a - rl);
    order_new[dst] = order[pos];
}

__global__ void k_nleft(const int64_t* __restrict__ L, const int64_t* __restrict__ seg, int nodes,
                        int64_t* __restrict__ nl) {
    const int k = blockIdx.x * blockDim.x + threadIdx.x;
    if (k < nodes) nl[k] = L[seg[k + 1]] - L[seg[k]];
}

__global__ void k_iota(uint32_t* o, int64_t n) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        o[i] = (uint32_t)i;
}

template <typename T>
void upload(DevBuf& b, const std::vector<T>& v, cudaStream_t s) {
    b.ensure(std::max<size_t>(v.size(), 1) * sizeof(T));
    if (!v.empty()) BLSH_CUDA(cudaMemcpyAsync(b.p, v.data(), v.size() * sizeof(T), cudaMemcpyHostToDevice, s));
}

}  // namespace

void build_rptree(blsh_index& ix, const float* Xs, uint32_t* order_dev, std::vector<int64_t>& seg,
                  cudaStream_t s) {
    const int64_t n = ix.n;
    const int d = ix.d, ds = ix.ds, G = ix.G;
    const int nn = std::max(G - 1, 1);
    k_iota<<<592, 256, 0, s>>>(order_dev, n);
    BLSH_LAUNCH_CHECK();
    seg.assign(2, 0);
    seg[1] = n;
    ix.theta_h.assign(nn, 0.0f);
    ix.ntype_h.assign(nn, 0);
    ix.mu_h.assign((size_t)nn * d, 0.0f);
    ix.diam2_h.assign(nn, 0.0);
    ix.da2_h.assign(nn, 0.0);
    ix.mu.alloc((size_t)nn * ds * sizeof(float));
    BLSH_CUDA(cudaMemsetAsync(ix.mu.p, 0, (size_t)nn * ds * sizeof(float), s));
    ix.theta.alloc(nn * sizeof(float));
    ix.ntype.alloc(nn * sizeof(int32_t));
    BLSH_CUDA(cudaMemsetAsync(ix.theta.p, 0, nn * sizeof(float), s));
    BLSH_CUDA(cudaMemsetAsync(ix.ntype.p, 0, nn * sizeof(int32_t), s));
    if (ix.depth == 0) return;

    DevBuf order2, vals, acc, left, L, tiles_d, chunks_d, part, csum, best_v, best_p, tile_off_d, tile_node_d,
        seg_d, nsz_d, chunk_off_d, vrow, sel, prefix, rank, hist, nl_d, diam_d, da_d, mnode_d, nodeids_d,
        theta_lvl;
    order2.alloc(std::max<int64_t>(n, 1) * sizeof(uint32_t));
    vals.alloc(std::max<int64_t>(n, 1) * sizeof(float));
    left.alloc(std::max<int64_t>(n, 1));
    L.alloc((std::max<int64_t>(n, 1) + 1) * sizeof(int64_t));
    if (ix.rp_rule == 0) acc.alloc(std::max<int64_t>(n, 1) * sizeof(double));
    ScanTemp scan;
    uint32_t* ord = order_dev;
    uint32_t* ord2 = order2.as<uint32_t>();
    const int m = std::max(1, ix.ek_iters);

    for (int lvl = 0; lvl < ix.depth; ++lvl) {
        const int nodes = 1 << lvl;
        const int node0 = nodes - 1;
        // work tables of this level
        std::vector<Tile> tiles;
        std::vector<Chunk> chunks;
        std::vector<int64_t> tile_off(nodes + 1, 0), chunk_off(nodes + 1, 0), nsz(nodes);
        std::vector<int32_t> tile_node(nodes);
        for (int k = 0; k < nodes; ++k) {
            const int64_t a = seg[k], e = seg[k + 1];
            nsz[k] = e - a;
            tile_node[k] = node0 + k;
            tile_off[k] = (int64_t)tiles.size();
            for (int64_t p = a; p < e; p += kTR) tiles.push_back(Tile{node0 + k, (int32_t)std::min<int64_t>(kTR, e - p), p});
            chunk_off[k] = (int64_t)chunks.size();
            for (int64_t p = a; p < e; p += kChunk) chunks.push_back(Chunk{node0 + k, (int32_t)std::min<int64_t>(kChunk, e - p), p});
        }
        tile_off[nodes] = (int64_t)tiles.size();
        chunk_off[nodes] = (int64_t)chunks.size();
        const int ntiles = (int)tiles.size(), nchunks = (int)chunks.size();
        upload(tiles_d, tiles, s);
        upload(chunks_d, chunks, s);
        upload(seg_d, seg, s);
        upload(nsz_d, nsz, s);
        upload(chunk_off_d, chunk_off, s);
        const Tile* T_d = tiles_d.as<Tile>();

        if (ix.rp_rule == 0 && ntiles > 0) {
            // ---- mean, Delta_A^2 (R7) ----
            part.ensure((size_t)std::max(nchunks, 1) * d * sizeof(double));
            dim3 g1(nchunks, (d + 127) / 128);
            k_colsum<<<g1, 128, 0, s>>>(Xs, ds, d, ord, chunks_d.as<Chunk>(), part.as<double>());
            BLSH_LAUNCH_CHECK();
            dim3 g2(nodes, (d + 127) / 128);
            k_mean_final<<<g2, 128, 0, s>>>(part.as<double>(), chunk_off_d.as<int64_t>(), nsz_d.as<int64_t>(),
                                            node0, d, ds, ix.mu.as<float>());
            BLSH_LAUNCH_CHECK();
            k_rowchain<RC_DIST><<<ntiles, kTR, 0, s>>>(Xs, ds, d, ord, T_d, ix.mu.as<float>(), nullptr, nullptr,
                                                       nullptr, vals.as<float>());
            BLSH_LAUNCH_CHECK();
            csum.ensure((size_t)std::max(nchunks, 1) * sizeof(double));
            k_chunksum<<<(nchunks + 127) / 128, 128, 0, s>>>(vals.as<float>(), chunks_d.as<Chunk>(), nchunks,
                                                             csum.as<double>());
            BLSH_LAUNCH_CHECK();
            da_d.ensure(nodes * sizeof(double));
            k_da_final<<<(nodes + 127) / 128, 128, 0, s>>>(csum.as<double>(), chunk_off_d.as<int64_t>(),
                                                           nsz_d.as<int64_t>(), nodes, da_d.as<double>());
            BLSH_LAUNCH_CHECK();
            // ---- approximate diameter (R6) ----
            best_v.ensure((size_t)ntiles * sizeof(double));
            best_p.ensure((size_t)ntiles * sizeof(int64_t));
            vrow.ensure((size_t)(node0 + nodes) * sizeof(uint32_t));
            sel.ensure((size_t)(node0 + nodes) * m * sizeof(uint32_t));
            // first member (lowest id) of every node is the start point
            std::vector<uint32_t> vr(node0 + nodes, 0);
            {
                std::vector<uint32_t> firsts(nodes, 0);
                // fetch order[seg[k]] for non-empty nodes
                for (int k = 0; k < nodes; ++k)
                    if (nsz[k] > 0)
                        BLSH_CUDA(cudaMemcpyAsync(&firsts[k], ord + seg[k], sizeof(uint32_t), cudaMemcpyDeviceToHost, s));
                BLSH_CUDA(cudaStreamSynchronize(s));
                for (int k = 0; k < nodes; ++k) vr[node0 + k] = firsts[k];
            }
            upload(vrow, vr, s);
            BLSH_CUDA(cudaMemsetAsync(acc.p, 0, (size_t)n * sizeof(double), s));
            std::vector<int32_t> mv(nodes);
            int mmax = 0;
            for (int k = 0; k < nodes; ++k) {
                mv[k] = (int)std::min<int64_t>(m, nsz[k]);
                mmax = std::max(mmax, mv[k]);
            }
            for (int it = -1; it + 1 < mmax; ++it) {
                // tiles of nodes that still select (it = -1: farthest from the first member)
                std::vector<Tile> at;
                std::vector<int64_t> at_off(1, 0);
                std::vector<int32_t> at_node;
                for (int k = 0; k < nodes; ++k) {
                    if (nsz[k] == 0 || it + 1 >= mv[k]) continue;
                    for (int64_t t = tile_off[k]; t < tile_off[k + 1]; ++t) at.push_back(tiles[t]);
                    at_off.push_back((int64_t)at.size());
                    at_node.push_back(node0 + k);
                }
                if (at.empty()) break;
                upload(tiles_d, at, s);
                upload(tile_off_d, at_off, s);
                upload(tile_node_d, at_node, s);
                const int nat = (int)at.size();
                k_rowchain<RC_DIST><<<nat, kTR, 0, s>>>(Xs, ds, d, ord, tiles_d.as<Tile>(), Xs, vrow.as<uint32_t>(),
                                                        nullptr, nullptr, vals.as<float>());
                BLSH_LAUNCH_CHECK();
                k_argmax_tiles<<<nat, kTR, 0, s>>>(vals.as<float>(), acc.as<double>(), it >= 0 ? 1 : 0,
                                                   tiles_d.as<Tile>(), best_v.as<double>(), best_p.as<int64_t>());
                BLSH_LAUNCH_CHECK();
                const int nan_ = (int)at_node.size();
                k_argmax_nodes<<<(nan_ + 127) / 128, 128, 0, s>>>(best_v.as<double>(), best_p.as<int64_t>(),
                                                                  tile_off_d.as<int64_t>(), tile_node_d.as<int32_t>(),
                                                                  nan_, ord, vrow.as<uint32_t>(), sel.as<uint32_t>(),
                                                                  it + 1, m);
                BLSH_LAUNCH_CHECK();
            }
            // pairs of selected points
            std::vector<int32_t> mn, nid;
            for (int k = 0; k < nodes; ++k)
                if (mv[k] >= 2) { mn.push_back(mv[k]); nid.push_back(node0 + k); }
            std::vector<double> diam(nodes, 0.0), da(nodes, 0.0);
            if (!mn.empty()) {
                upload(mnode_d, mn, s);
                upload(nodeids_d, nid, s);
                diam_d.ensure(mn.size() * sizeof(double));
                k_pairmax<<<(unsigned)mn.size(), 256, 0, s>>>(Xs, ds, d, sel.as<uint32_t>(), mnode_d.as<int32_t>(),
                                                              nodeids_d.as<int32_t>(), m, diam_d.as<double>());
                BLSH_LAUNCH_CHECK();
                std::vector<double> dv(mn.size());
                BLSH_CUDA(cudaMemcpyAsync(dv.data(), diam_d.p, dv.size() * sizeof(double), cudaMemcpyDeviceToHost, s));
                BLSH_CUDA(cudaStreamSynchronize(s));
                for (size_t i = 0; i < nid.size(); ++i) diam[nid[i] - node0] = dv[i];
            }
            BLSH_CUDA(cudaMemcpyAsync(da.data(), da_d.p, nodes * sizeof(double), cudaMemcpyDeviceToHost, s));
            BLSH_CUDA(cudaStreamSynchronize(s));
            for (int k = 0; k < nodes; ++k) {
                ix.diam2_h[node0 + k] = diam[k];
                ix.da2_h[node0 + k] = da[k];
                const double rhs = ix.rp_mean_c * da[k];   // compiled without contraction
                ix.ntype_h[node0 + k] = (nsz[k] == 0 || diam[k] <= rhs) ? 0 : 1;
            }
            BLSH_CUDA(cudaMemcpyAsync(ix.ntype.as<int32_t>() + node0, ix.ntype_h.data() + node0,
                                      nodes * sizeof(int32_t), cudaMemcpyHostToDevice, s));
            upload(tiles_d, tiles, s);   // restore the full tile table
        }
        if (ntiles > 0) {
            // ---- split values, exact lower median (R5) ----
            k_rowchain<RC_SPLIT><<<ntiles, kTR, 0, s>>>(Xs, ds, d, ord, tiles_d.as<Tile>(), ix.dirs.as<float>(),
                                                        nullptr, ix.ntype.as<int32_t>(), ix.mu.as<float>(),
                                                        vals.as<float>());
            BLSH_LAUNCH_CHECK();
            prefix.ensure(nodes * sizeof(uint32_t));
            rank.ensure(nodes * sizeof(int64_t));
            hist.ensure((size_t)nodes * 256 * sizeof(uint32_t));
            BLSH_CUDA(cudaMemsetAsync(prefix.p, 0, nodes * sizeof(uint32_t), s));
            BLSH_CUDA(cudaMemsetAsync(hist.p, 0, (size_t)nodes * 256 * sizeof(uint32_t), s));
            std::vector<int64_t> rk(nodes);
            for (int k = 0; k < nodes; ++k) rk[k] = nsz[k] > 0 ? (nsz[k] - 1) / 2 : 0;
            upload(rank, rk, s);
            for (int shift = 24; shift >= 0; shift -= 8) {
                k_sel_hist<<<ntiles, kTR, 0, s>>>(vals.as<float>(), tiles_d.as<Tile>(), node0, prefix.as<uint32_t>(),
                                                  shift, hist.as<uint32_t>());
                BLSH_LAUNCH_CHECK();
                k_sel_pick<<<nodes, 256, 0, s>>>(hist.as<uint32_t>(), prefix.as<uint32_t>(), rank.as<int64_t>(),
                                                 nsz_d.as<int64_t>(), shift);
                BLSH_LAUNCH_CHECK();
            }
            theta_lvl.ensure(nodes * sizeof(float));
            k_theta<<<(nodes + 127) / 128, 128, 0, s>>>(prefix.as<uint32_t>(), nsz_d.as<int64_t>(), nodes,
                                                       theta_lvl.as<float>());
            BLSH_LAUNCH_CHECK();
            std::vector<float> th(nodes);
            BLSH_CUDA(cudaMemcpyAsync(th.data(), theta_lvl.p, nodes * sizeof(float), cudaMemcpyDeviceToHost, s));
            BLSH_CUDA(cudaStreamSynchronize(s));
            if (ix.rp_rule == 1 && ix.rp_max_jitter != 0.0) {
                // RP-tree max jitter (R4): farthest point y from the first member x0
                std::vector<uint32_t> vr(node0 + nodes, 0);
                for (int k = 0; k < nodes; ++k)
                    if (nsz[k] > 0)
                        BLSH_CUDA(cudaMemcpyAsync(&vr[node0 + k], ord + seg[k], sizeof(uint32_t), cudaMemcpyDeviceToHost, s));
                BLSH_CUDA(cudaStreamSynchronize(s));
                upload(vrow, vr, s);
                k_rowchain<RC_DIST><<<ntiles, kTR, 0, s>>>(Xs, ds, d, ord, tiles_d.as<Tile>(), Xs, vrow.as<uint32_t>(),
                                                           nullptr, nullptr, vals.as<float>());
                BLSH_LAUNCH_CHECK();
                best_v.ensure((size_t)ntiles * sizeof(double));
                best_p.ensure((size_t)ntiles * sizeof(int64_t));
                k_argmax_tiles<<<ntiles, kTR, 0, s>>>(vals.as<float>(), nullptr, 0, tiles_d.as<Tile>(),
                                                      best_v.as<double>(), best_p.as<int64_t>());
                BLSH_LAUNCH_CHECK();
                std::vector<double> bv(ntiles);
                BLSH_CUDA(cudaMemcpyAsync(bv.data(), best_v.p, ntiles * sizeof(double), cudaMemcpyDeviceToHost, s));
                BLSH_CUDA(cudaStreamSynchronize(s));
                for (int k = 0; k < nodes; ++k) {
                    if (nsz[k] == 0) continue;
                    double bd = -1.0;
                    for (int64_t t = tile_off[k]; t < tile_off[k + 1]; ++t) bd = std::max(bd, bv[t]);
                    const double delta = (2.0 * ix.jit_h[node0 + k] - 1.0) * ix.rp_max_jitter * std::sqrt(bd) /
                                         std::sqrt((double)d);
                    th[k] = (float)((double)th[k] + delta);
                }
                // the split values were overwritten: recompute them
                k_rowchain<RC_SPLIT><<<ntiles, kTR, 0, s>>>(Xs, ds, d, ord, tiles_d.as<Tile>(), ix.dirs.as<float>(),
                                                            nullptr, ix.ntype.as<int32_t>(), ix.mu.as<float>(),
                                                            vals.as<float>());
                BLSH_LAUNCH_CHECK();
            }
            for (int k = 0; k < nodes; ++k) ix.theta_h[node0 + k] = th[k];
            BLSH_CUDA(cudaMemcpyAsync(ix.theta.as<float>() + node0, th.data(), nodes * sizeof(float),
                                      cudaMemcpyHostToDevice, s));
            // ---- stable partition ----
            k_left_flags<<<ntiles, kTR, 0, s>>>(vals.as<float>(), tiles_d.as<Tile>(), ix.theta.as<float>(),
                                                left.as<uint8_t>());
            BLSH_LAUNCH_CHECK();
        }
        if (n > 0) {
            if (ntiles == 0) BLSH_CUDA(cudaMemsetAsync(left.p, 0, n, s));
            scan_exclusive_u8(left.as<uint8_t>(), L.as<int64_t>(), n, scan, s);
            if (ntiles > 0) {
                k_partition<<<ntiles, kTR, 0, s>>>(ord, left.as<uint8_t>(), L.as<int64_t>(), tiles_d.as<Tile>(),
                                                   seg_d.as<int64_t>(), node0, ord2);
                BLSH_LAUNCH_CHECK();
            }
            nl_d.ensure(nodes * sizeof(int64_t));
            k_nleft<<<(nodes + 127) / 128, 128, 0, s>>>(L.as<int64_t>(), seg_d.as<int64_t>(), nodes, nl_d.as<int64_t>());
            BLSH_LAUNCH_CHECK();
        }
        std::vector<int64_t> nl(nodes, 0);
        if (n > 0) {
            BLSH_CUDA(cudaMemcpyAsync(nl.data(), nl_d.p, nodes * sizeof(int64_t), cudaMemcpyDeviceToHost, s));
            BLSH_CUDA(cudaStreamSynchronize(s));
        }
        std::vector<int64_t> nseg(2 * nodes + 1);
        for (int k = 0; k < nodes; ++k) {
            nseg[2 * k] = seg[k];
            nseg[2 * k + 1] = seg[k] + nl[k];
        }
        nseg[2 * nodes] = n;
        seg.swap(nseg);
        if (ntiles > 0) std::swap(ord, ord2);
    }
    if (ord != order_dev) BLSH_CUDA(cudaMemcpyAsync(order_dev, ord, n * sizeof(uint32_t), cudaMemcpyDeviceToDevice, s));
    // host copies of mu for export
    std::vector<float> mup((size_t)nn * ds);
    BLSH_CUDA(cudaMemcpyAsync(mup.data(), ix.mu.p, mup.size() * sizeof(float), cudaMemcpyDeviceToHost, s));
    BLSH_CUDA(cudaStreamSynchronize(s));
    for (int v = 0; v < nn; ++v)
        for (int j = 0; j < d; ++j) ix.mu_h[(size_t)v * d + j] = mup[(size_t)v * ds + j];
}

// Per-leaf spread for the W rule of P:107 (reading R29): Delta_A^2(g) =
// 2 sum dist2c(x, mu_g) / |g| over the leaf's members in ascending id, with the
// same R7 reductions (chunks of 4096, fp64, in order) as the tree's nodes.
void leaf_spread(const blsh_index& ix, const float* Xs, const uint32_t* order, const std::vector<int64_t>& seg,
                 std::vector<double>& da2_out, cudaStream_t s) {
    const int G = ix.G, d = ix.d, ds = ix.ds;
    da2_out.assign(G, 0.0);
    std::vector<Tile> tiles;
    std::vector<Chunk> chunks;
    std::vector<int64_t> chunk_off(G + 1, 0), nsz(G);
    for (int k = 0; k < G; ++k) {
        const int64_t a = seg[k], e = seg[k + 1];
        nsz[k] = e - a;
        for (int64_t p = a; p < e; p += kTR) tiles.push_back(Tile{k, (int32_t)std::min<int64_t>(kTR, e - p), p});
        chunk_off[k] = (int64_t)chunks.size();
        for (int64_t p = a; p < e; p += kChunk) chunks.push_back(Chunk{k, (int32_t)std::min<int64_t>(kChunk, e - p), p});
    }
    chunk_off[G] = (int64_t)chunks.size();
    const int ntiles = (int)tiles.size(), nchunks = (int)chunks.size();
    if (ntiles == 0) return;
    DevBuf tiles_d, chunks_d, chunk_off_d, nsz_d, part, mu, vals, csum, da;
    upload(tiles_d, tiles, s);
    upload(chunks_d, chunks, s);
    upload(chunk_off_d, chunk_off, s);
    upload(nsz_d, nsz, s);
    part.alloc((size_t)nchunks * d * sizeof(double));
    mu.alloc((size_t)G * ds * sizeof(float));
    BLSH_CUDA(cudaMemsetAsync(mu.p, 0, (size_t)G * ds * sizeof(float), s));
    vals.alloc((size_t)std::max<int64_t>(ix.n, 1) * sizeof(float));
    csum.alloc((size_t)nchunks * sizeof(double));
    da.alloc((size_t)G * sizeof(double));
    k_colsum<<<dim3(nchunks, (d + 127) / 128), 128, 0, s>>>(Xs, ds, d, order, chunks_d.as<Chunk>(), part.as<double>());
    BLSH_LAUNCH_CHECK();
    k_mean_final<<<dim3(G, (d + 127) / 128), 128, 0, s>>>(part.as<double>(), chunk_off_d.as<int64_t>(),
                                                          nsz_d.as<int64_t>(), 0, d, ds, mu.as<float>());
    BLSH_LAUNCH_CHECK();
    k_rowchain<RC_DIST><<<ntiles, kTR, 0, s>>>(Xs, ds, d, order, tiles_d.as<Tile>(), mu.as<float>(), nullptr, nullptr,
                                               nullptr, vals.as<float>());
    BLSH_LAUNCH_CHECK();
    k_chunksum<<<(nchunks + 127) / 128, 128, 0, s>>>(vals.as<float>(), chunks_d.as<Chunk>(), nchunks, csum.as<double>());
    BLSH_LAUNCH_CHECK();
    k_da_final<<<(G + 127) / 128, 128, 0, s>>>(csum.as<double>(), chunk_off_d.as<int64_t>(), nsz_d.as<int64_t>(), G,
                                               da.as<double>());
    BLSH_LAUNCH_CHECK();
    BLSH_CUDA(cudaMemcpyAsync(da2_out.data(), da.p, G * sizeof(double), cudaMemcpyDeviceToHost, s));
    BLSH_CUDA(cudaStreamSynchronize(s));
}

}  // namespace blsh
