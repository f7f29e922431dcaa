// api.cu -- the C ABI (include/blsh.h): argument checks, memory, orchestration
// of the build (b1-b4) and of the query hot path (a1-a6).
#include <algorithm>
#include <chrono>
#include <cmath>
#include <cstdlib>
#include <cstring>
#include <string>

#include "internal.cuh"
#include "query_kernels.cuh"

namespace {

thread_local std::string g_last_error;

blsh_status fail(blsh_status c, const std::string& m) {
    g_last_error = m;
    return c;
}

bool is_device_ptr(const void* p) {
    if (!p) return false;
    cudaPointerAttributes at{};
    if (cudaPointerGetAttributes(&at, p) != cudaSuccess) {
        cudaGetLastError();
        return false;
    }
    return at.type == cudaMemoryTypeDevice || at.type == cudaMemoryTypeManaged;
}

template <typename F>
blsh_status guarded(F&& f) {
    try {
        f();
        return BLSH_OK;
    } catch (const blsh::Error& e) {
        return fail(e.code, e.what());
    } catch (const std::bad_alloc&) {
        return fail(BLSH_ERR_OOM, "host allocation failed");
    } catch (const std::exception& e) {
        return fail(BLSH_ERR_CUDA, e.what());
    }
}

__global__ void k_point_leaf(const uint32_t* __restrict__ order, const int64_t* __restrict__ seg, int G,
                             int32_t* __restrict__ pt_leaf) {
    const int g = blockIdx.y;
    if (g >= G) return;
    for (int64_t p = seg[g] + blockIdx.x * (int64_t)blockDim.x + threadIdx.x; p < seg[g + 1];
         p += (int64_t)gridDim.x * blockDim.x)
        pt_leaf[order[p]] = g;
}

__global__ void k_point_key(const unsigned long long* __restrict__ hi, const unsigned long long* __restrict__ lo,
                            const uint32_t* __restrict__ id, int64_t n, blsh::Key128* __restrict__ pt_key) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        pt_key[id[i]] = blsh::Key128{hi[i], lo[i]};
}

int64_t ipow3(int M) {
    int64_t p = 1;
    for (int i = 0; i < M; ++i) p *= 3;
    return p;
}

}  // namespace

extern "C" {

void blsh_build_params_default(blsh_build_params* p) {
    if (!p) return;
    std::memset(p, 0, sizeof(*p));
    p->n_leaves = 1;
    p->rp_rule = 0;
    p->rp_mean_c = 10.0;
    p->rp_max_jitter = 0.0;
    p->ek_iters = 40;
    p->M = 8;
    p->quantizer = 0;
    p->W = 4.0f;
    p->W_leaf = nullptr;
    p->seed = 42;
    p->rank = 0;
    p->world = 1;
    p->stream = nullptr;
    p->keep_stages = 0;
    p->n_tables = 1;
}

void blsh_query_params_default(blsh_query_params* p) {
    if (!p) return;
    std::memset(p, 0, sizeof(*p));
    p->probe = 0;
    p->n_probes = 1;
    p->hierarchy = 0;
    p->hier_step_bits = 0;
    p->min_cand = 0;
    p->stream = nullptr;
    p->keep_stages = 0;
    p->timing = 0;
    p->global_base = nullptr;
}

const char* blsh_last_error(void) { return g_last_error.c_str(); }

void blsh_free(blsh_index* idx) {
    if (!idx) return;
    for (auto& e : idx->ev)
        if (e) cudaEventDestroy(e);
    delete idx;
}

blsh_status blsh_build(const float* X, int64_t n, int32_t d, const blsh_build_params* p, blsh_index** out) {
    if (!out) return fail(BLSH_ERR_INVALID, "out is NULL");
    *out = nullptr;
    if (!p) return fail(BLSH_ERR_INVALID, "params is NULL");
    if (n < 0 || n >= (int64_t(1) << 31)) return fail(BLSH_ERR_INVALID, "n must be in [0, 2^31)");
    if (n > 0 && !X) return fail(BLSH_ERR_INVALID, "X is NULL");
    if (d < 1 || d > 1024) return fail(BLSH_ERR_INVALID, "d must be in [1, 1024]");
    const int G = p->n_leaves;
    if (G < 1 || G > 4096 || (G & (G - 1))) return fail(BLSH_ERR_INVALID, "n_leaves must be a power of two in [1, 4096]");
    if (p->M < 1 || p->M > 16) return fail(BLSH_ERR_INVALID, "M must be in [1, 16]");
    if (p->quantizer != 0 && p->quantizer != 1) return fail(BLSH_ERR_INVALID, "quantizer must be 0 or 1");
    if (p->quantizer == 1 && p->M != 8 && p->M != 16)
        return fail(BLSH_ERR_INVALID, "E8 quantizer needs M = 8 or 16 (ceil(M/8) E8 blocks, P:175)");
    if (!(p->W > 0.0f) || !std::isfinite(p->W)) return fail(BLSH_ERR_INVALID, "W must be > 0");
    if (p->rp_rule != 0 && p->rp_rule != 1) return fail(BLSH_ERR_INVALID, "rp_rule must be 0 or 1");
    if (p->ek_iters < 1) return fail(BLSH_ERR_INVALID, "ek_iters must be >= 1");
    if (p->world < 1 || p->rank < 0 || p->rank >= p->world)
        return fail(BLSH_ERR_INVALID, "rank/world must satisfy 0 <= rank < world");
    if (p->leaf_split) {
        if (p->leaf_split[0] != 0 || p->leaf_split[p->world] != G)
            return fail(BLSH_ERR_INVALID, "leaf_split must start at 0 and end at n_leaves");
        for (int r = 0; r < p->world; ++r)
            if (p->leaf_split[r + 1] < p->leaf_split[r]) return fail(BLSH_ERR_INVALID, "leaf_split must be non-decreasing");
    } else if (G % p->world != 0) {
        return fail(BLSH_ERR_INVALID, "world must divide n_leaves (or pass leaf_split)");
    }
    if (p->n_tables < 1 || p->n_tables > 64) return fail(BLSH_ERR_INVALID, "n_tables must be in [1, 64]");
    if (p->W_rule != 0 && p->W_rule != 1) return fail(BLSH_ERR_INVALID, "W_rule must be 0 or 1");
    if (p->W_rule == 1 && p->W_leaf) return fail(BLSH_ERR_INVALID, "W_rule = 1 derives the per-leaf widths (no W_leaf)");
    if (p->W_leaf)
        for (int g = 0; g < G; ++g)
            if (!(p->W_leaf[g] > 0.0f) || !std::isfinite(p->W_leaf[g])) return fail(BLSH_ERR_INVALID, "W_leaf must be > 0");
    auto t0 = std::chrono::steady_clock::now();
    blsh_index* ix = new (std::nothrow) blsh_index();
    if (!ix) return fail(BLSH_ERR_OOM, "host allocation failed");
    cudaStream_t s = (cudaStream_t)p->stream;
    blsh_status st = guarded([&] {
        blsh::upload_e8_roots();
        ix->n = n;
        ix->d = d;
        ix->ds = (d + 3) & ~3;
        ix->G = G;
        ix->M = p->M;
        ix->B = blsh::bits_per_coord(p->M);
        ix->quantizer = p->quantizer;
        ix->rp_rule = p->rp_rule;
        ix->rp_mean_c = p->rp_mean_c;
        ix->rp_max_jitter = p->rp_max_jitter;
        ix->ek_iters = p->ek_iters;
        ix->seed = p->seed;
        ix->rank = p->rank;
        ix->world = p->world;
        ix->leaf_lo = p->leaf_split ? p->leaf_split[p->rank] : p->rank * (G / p->world);
        ix->leaf_hi = p->leaf_split ? p->leaf_split[p->rank + 1] : (p->rank + 1) * (G / p->world);
        int depth = 0;
        while ((1 << depth) < G) ++depth;
        ix->depth = depth;
        const int ds = ix->ds, M = ix->M, nn = std::max(G - 1, 1);
        // b1: parameters (host, R2)
        ix->W_h.resize(G);
        for (int g = 0; g < G; ++g) ix->W_h[g] = p->W_leaf ? p->W_leaf[g] : p->W;
        ix->A_h.assign((size_t)G * M * d, 0.0f);
        ix->b_h.assign((size_t)G * M, 0.0f);
        ix->dirs_h.assign((size_t)nn * d, 0.0f);
        ix->jit_h.assign(nn, 0.0);
        blsh::gen_params(p->seed, G, M, d, ix->W_h.data(), ix->A_h.data(), ix->b_h.data(), ix->dirs_h.data(),
                         ix->jit_h.data());
        ix->A.alloc(ix->A_h.size() * sizeof(float));
        ix->b.alloc(ix->b_h.size() * sizeof(float));
        ix->W.alloc(G * sizeof(float));
        BLSH_CUDA(cudaMemcpyAsync(ix->A.p, ix->A_h.data(), ix->A_h.size() * sizeof(float), cudaMemcpyHostToDevice, s));
        BLSH_CUDA(cudaMemcpyAsync(ix->b.p, ix->b_h.data(), ix->b_h.size() * sizeof(float), cudaMemcpyHostToDevice, s));
        BLSH_CUDA(cudaMemcpyAsync(ix->W.p, ix->W_h.data(), G * sizeof(float), cudaMemcpyHostToDevice, s));
        ix->dirs.alloc((size_t)nn * ds * sizeof(float));
        BLSH_CUDA(cudaMemsetAsync(ix->dirs.p, 0, (size_t)nn * ds * sizeof(float), s));
        if (G > 1)
            BLSH_CUDA(cudaMemcpy2DAsync(ix->dirs.p, ds * sizeof(float), ix->dirs_h.data(), d * sizeof(float),
                                        d * sizeof(float), G - 1, cudaMemcpyHostToDevice, s));
        // data in the padded row layout
        blsh::DevBuf Xs;
        Xs.alloc((size_t)std::max<int64_t>(n, 1) * ds * sizeof(float));
        if (ds != d) BLSH_CUDA(cudaMemsetAsync(Xs.p, 0, (size_t)std::max<int64_t>(n, 1) * ds * sizeof(float), s));
        if (n > 0)
            BLSH_CUDA(cudaMemcpy2DAsync(Xs.p, ds * sizeof(float), X, d * sizeof(float), d * sizeof(float), n,
                                        cudaMemcpyDefault, s));
        // b2: RP-tree
        blsh::DevBuf order;
        order.alloc((size_t)std::max<int64_t>(n, 1) * sizeof(uint32_t));
        std::vector<int64_t> seg;
        blsh::build_rptree(*ix, Xs.as<float>(), order.as<uint32_t>(), seg, s);
        if (p->W_rule == 1) {
            // P:107 / R29: per-leaf widths from the leaves' spread, then (a, b) redrawn with them
            // (b = W_g U depends on W_g; a and the tree do not)
            blsh::leaf_spread(*ix, Xs.as<float>(), order.as<uint32_t>(), seg, ix->leaf_da2_h, s);
            std::vector<double> srt(ix->leaf_da2_h);
            std::sort(srt.begin(), srt.end());
            const double med = srt[(G - 1) / 2];
            for (int g = 0; g < G; ++g) {
                const double dg = ix->leaf_da2_h[g];
                ix->W_h[g] = (dg > 0.0 && med > 0.0) ? (float)((double)p->W * std::sqrt(dg / med)) : p->W;
                if (!(ix->W_h[g] > 0.0f) || !std::isfinite(ix->W_h[g])) ix->W_h[g] = p->W;
            }
            blsh::gen_params(p->seed, G, M, d, ix->W_h.data(), ix->A_h.data(), ix->b_h.data(), ix->dirs_h.data(),
                             ix->jit_h.data());
            BLSH_CUDA(cudaMemcpyAsync(ix->A.p, ix->A_h.data(), ix->A_h.size() * sizeof(float), cudaMemcpyHostToDevice, s));
            BLSH_CUDA(cudaMemcpyAsync(ix->b.p, ix->b_h.data(), ix->b_h.size() * sizeof(float), cudaMemcpyHostToDevice, s));
            BLSH_CUDA(cudaMemcpyAsync(ix->W.p, ix->W_h.data(), G * sizeof(float), cudaMemcpyHostToDevice, s));
            BLSH_CUDA(cudaStreamSynchronize(s));
        }
        const int64_t pos_lo = seg[ix->leaf_lo], pos_hi = seg[ix->leaf_hi];
        const int64_t no = pos_hi - pos_lo;
        ix->n_owned = no;
        // b3: hash owned points
        blsh::SortBufs sb;
        for (int i = 0; i < 2; ++i) {
            sb.hi[i].alloc((size_t)std::max<int64_t>(no, 1) * 8);
            sb.lo[i].alloc((size_t)std::max<int64_t>(no, 1) * 8);
            sb.leaf[i].alloc((size_t)std::max<int64_t>(no, 1) * 4);
            sb.id[i].alloc((size_t)std::max<int64_t>(no, 1) * 4);
        }
        int32_t* code_out = nullptr;
        if (p->keep_stages) {
            ix->pt_code.alloc((size_t)std::max<int64_t>(n, 1) * M * sizeof(int32_t));
            BLSH_CUDA(cudaMemsetAsync(ix->pt_code.p, 0, (size_t)std::max<int64_t>(n, 1) * M * sizeof(int32_t), s));
            code_out = ix->pt_code.as<int32_t>();
        }
        const bool ok = blsh::hash_points(*ix, Xs.as<float>(), order.as<uint32_t>(), seg, pos_lo, pos_hi,
                                          sb.hi[0].as<unsigned long long>(), sb.lo[0].as<unsigned long long>(),
                                          sb.leaf[0].as<uint32_t>(), sb.id[0].as<uint32_t>(), code_out, s);
        if (!ok) throw blsh::Error(BLSH_ERR_RANGE, "a data point's code leaves the Morton range (decrease M or increase W)");
        if (p->keep_stages) {
            ix->pt_leaf.alloc((size_t)std::max<int64_t>(n, 1) * sizeof(int32_t));
            ix->pt_key.alloc((size_t)std::max<int64_t>(n, 1) * sizeof(blsh::Key128));
            BLSH_CUDA(cudaMemsetAsync(ix->pt_key.p, 0, (size_t)std::max<int64_t>(n, 1) * sizeof(blsh::Key128), s));
            blsh::DevBuf seg_d;
            seg_d.alloc(seg.size() * sizeof(int64_t));
            BLSH_CUDA(cudaMemcpyAsync(seg_d.p, seg.data(), seg.size() * sizeof(int64_t), cudaMemcpyHostToDevice, s));
            dim3 g(64, G);
            k_point_leaf<<<g, 256, 0, s>>>(order.as<uint32_t>(), seg_d.as<int64_t>(), G, ix->pt_leaf.as<int32_t>());
            BLSH_LAUNCH_CHECK();
            if (no > 0) {
                k_point_key<<<592, 256, 0, s>>>(sb.hi[0].as<unsigned long long>(), sb.lo[0].as<unsigned long long>(),
                                                sb.id[0].as<uint32_t>(), no, ix->pt_key.as<blsh::Key128>());
                BLSH_LAUNCH_CHECK();
            }
            BLSH_CUDA(cudaStreamSynchronize(s));
            ix->has_pt = true;
        }
        // b4: sort + table
        int passes = 0;
        const int cur = blsh::radix_sort_entries(sb, no, s, &passes);
        blsh::build_table(*ix, Xs.as<float>(), sb.hi[cur].as<unsigned long long>(), sb.lo[cur].as<unsigned long long>(),
                          sb.leaf[cur].as<uint32_t>(), sb.id[cur].as<uint32_t>(), no, sb.scan, s);
        blsh::build_screen_rows(*ix, s);   // the short-list screen's fp16 residual rows (resid.cu)
        BLSH_CUDA(cudaStreamSynchronize(s));
        // leaves as table position ranges (the same in every table: entries sort by leaf first)
        ix->leaf_pos_h.assign(G + 1, 0);
        ix->max_leaf_rows = 0;
        for (int g = 0; g <= G; ++g)
            ix->leaf_pos_h[g] = std::min<int64_t>(no, std::max<int64_t>(0, seg[g] - pos_lo));
        for (int g = ix->leaf_lo; g < ix->leaf_hi; ++g)
            ix->max_leaf_rows = std::max<int64_t>(ix->max_leaf_rows, ix->leaf_pos_h[g + 1] - ix->leaf_pos_h[g]);
        ix->leaf_pos.alloc((G + 1) * sizeof(int64_t));
        BLSH_CUDA(cudaMemcpyAsync(ix->leaf_pos.p, ix->leaf_pos_h.data(), (G + 1) * sizeof(int64_t),
                                  cudaMemcpyHostToDevice, s));
        // E8 index: the code hierarchy of P:162-173 over the primary table's buckets
        if (ix->quantizer == 1) blsh::build_e8_hierarchy(*ix, s);
        // tables 1..L-1: own (a, b), same tree and rows
        ix->L = p->n_tables;
        std::vector<const uint32_t*> tab_pos(ix->L, nullptr);
        if (ix->L > 1) {
            blsh::DevBuf inv0;
            inv0.alloc((size_t)std::max<int64_t>(n, 1) * sizeof(uint32_t));
            blsh::invert_perm(ix->perm.as<uint32_t>(), no, inv0.as<uint32_t>(), s);
            for (int l = 1; l < ix->L; ++l) {
                auto t = std::make_unique<blsh::ExtraTable>();
                t->A_h.assign((size_t)G * M * d, 0.0f);
                t->b_h.assign((size_t)G * M, 0.0f);
                blsh::gen_table_params(p->seed, l, G, M, d, ix->W_h.data(), t->A_h.data(), t->b_h.data());
                t->A.alloc(t->A_h.size() * sizeof(float));
                t->b.alloc(t->b_h.size() * sizeof(float));
                BLSH_CUDA(cudaMemcpyAsync(t->A.p, t->A_h.data(), t->A_h.size() * sizeof(float), cudaMemcpyHostToDevice, s));
                BLSH_CUDA(cudaMemcpyAsync(t->b.p, t->b_h.data(), t->b_h.size() * sizeof(float), cudaMemcpyHostToDevice, s));
                const bool okl = blsh::hash_points(*ix, Xs.as<float>(), order.as<uint32_t>(), seg, pos_lo, pos_hi,
                                                   sb.hi[0].as<unsigned long long>(), sb.lo[0].as<unsigned long long>(),
                                                   sb.leaf[0].as<uint32_t>(), sb.id[0].as<uint32_t>(), nullptr, s,
                                                   t->A.as<float>(), t->b.as<float>());
                if (!okl) throw blsh::Error(BLSH_ERR_RANGE, "a data point's code leaves the Morton range (decrease M or increase W)");
                const int cl = blsh::radix_sort_entries(sb, no, s, &passes);
                blsh::build_extra_table(*ix, *t, sb.hi[cl].as<unsigned long long>(), sb.lo[cl].as<unsigned long long>(),
                                        sb.leaf[cl].as<uint32_t>(), sb.id[cl].as<uint32_t>(), inv0.as<uint32_t>(), no,
                                        sb.scan, s);
                tab_pos[l] = t->pos.as<uint32_t>();
                ix->xt.push_back(std::move(t));
            }
        }
        ix->tab_pos.alloc(ix->L * sizeof(const uint32_t*));
        BLSH_CUDA(cudaMemcpyAsync(ix->tab_pos.p, tab_pos.data(), ix->L * sizeof(const uint32_t*), cudaMemcpyHostToDevice, s));
        BLSH_CUDA(cudaStreamSynchronize(s));
        for (auto& e : ix->ev) BLSH_CUDA(cudaEventCreate(&e));
    });
    if (st != BLSH_OK) {
        delete ix;
        return st;
    }
    ix->build_ms = std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
    *out = ix;
    return BLSH_OK;
}

}  // extern "C"

namespace blsh {

static void run_query_core(const blsh_index& ix, const float* Q, bool q_host, int64_t nq, int k,
                           const blsh_query_params& p, int64_t* out_ids, float* out_d2,
                           unsigned long long* out_packed, int64_t* out_ncand, bool out_host, int64_t* out_base,
                           bool capture = false);
static bool query_graph(const blsh_index& ix, const float* Q, int64_t nq, int k, const blsh_query_params& p,
                        int64_t* out_ids, float* out_d2, int64_t* out_ncand);

// Small batches (<= small_batch_limit() queries on the warp short-list, whose plan needs no host
// round trip): the whole call -- route, hash, probes, plan, short-list, merge, ~17 launches whose
// host-side issue dominated the latency (GPU span 0.21 ms for one query, r02at) -- is captured
// once per (shape, parameters, workspace) into a CUDA graph on a private stream and replayed on the
// caller's stream: copy the batch into the graph's input buffer, launch, copy the answers out.
// The first call of a shape runs normally (allocating every workspace buffer), then captures.
// Results are those of run_query_core (the same kernels on the same inputs).  BLSH_GRAPH=0
// disables it (experiments).
static bool query_graph(const blsh_index& ix, const float* Q, int64_t nq, int k, const blsh_query_params& p,
                        int64_t* out_ids, float* out_d2, int64_t* out_ncand) {
    static const bool enabled = [] {
        const char* e = std::getenv("BLSH_GRAPH");
        return !(e && e[0] == '0');
    }();
    if (!enabled || nq <= 0 || nq > small_batch_limit() || p.keep_stages || p.timing || p.global_base || ix.L > 1 ||
        (p.hierarchy == 1 && ix.quantizer == 1) || shortlist_kind(nq, ix.ds, ix.dr, p.n_probes, k) != 0)
        return false;
    QueryWork& w = ix.qw;
    cudaStream_t s = (cudaStream_t)p.stream;
    const size_t qbytes = (size_t)nq * ix.d * sizeof(float);
    const size_t ib = ((size_t)nq * k * 8 + 255) & ~size_t(255), db = ((size_t)nq * k * 4 + 255) & ~size_t(255);
    w.g_q.ensure(qbytes);
    w.g_out.ensure(ib + db + (size_t)nq * 8);
    const float* gq = w.g_q.as<float>();
    int64_t* gi = w.g_out.as<int64_t>();
    float* gd = reinterpret_cast<float*>(w.g_out.as<char>() + ib);
    int64_t* gn = reinterpret_cast<int64_t*>(w.g_out.as<char>() + ib + db);
    BLSH_CUDA(cudaMemcpyAsync(w.g_q.p, Q, qbytes, cudaMemcpyDeviceToDevice, s));
    auto key_of = [&](QueryWork::GraphEntry& e) {
        e.nq = nq; e.min_cand = p.min_cand; e.k = k; e.T = p.n_probes; e.probe = p.probe; e.hierarchy = p.hierarchy;
        e.hstep = p.hier_step_bits; e.cperturb = p.curve_perturb; e.msb_min = p.msb_min;
        const DevBuf* b[6] = {&w.arena, &w.partials, &w.scan.blocks, &w.g_q, &w.g_out, &w.listbuf};
        for (int i = 0; i < 6; ++i) { e.bufs[i] = b[i]->p; e.sizes[i] = b[i]->bytes; }
    };
    auto same = [](const QueryWork::GraphEntry& a, const QueryWork::GraphEntry& b) {
        if (a.nq != b.nq || a.min_cand != b.min_cand || a.k != b.k || a.T != b.T || a.probe != b.probe ||
            a.hierarchy != b.hierarchy || a.hstep != b.hstep || a.cperturb != b.cperturb || a.msb_min != b.msb_min)
            return false;
        for (int i = 0; i < 6; ++i)
            if (a.bufs[i] != b.bufs[i] || a.sizes[i] != b.sizes[i]) return false;
        return true;
    };
    QueryWork::GraphEntry key{};
    key_of(key);
    QueryWork::GraphEntry* hit = nullptr;
    for (auto& e : w.graphs)
        if (same(e, key)) { hit = &e; break; }
    if (!hit) {
        // run it once for real (allocates the workspace, gives this call's answers), then capture
        run_query_core(ix, gq, false, nq, k, p, gi, gd, nullptr, gn, false, nullptr);
        QueryWork::GraphEntry e{};
        key_of(e);
        e.stats = ix.stats;
        if (!w.cap) BLSH_CUDA(cudaStreamCreateWithFlags(&w.cap, cudaStreamNonBlocking));
        blsh_query_params pc = p;
        pc.stream = w.cap;
        cudaGraph_t g = nullptr;
        BLSH_CUDA(cudaStreamBeginCapture(w.cap, cudaStreamCaptureModeRelaxed));
        try {
            run_query_core(ix, gq, false, nq, k, pc, gi, gd, nullptr, gn, false, nullptr, true);
        } catch (...) {
            cudaStreamEndCapture(w.cap, &g);
            if (g) cudaGraphDestroy(g);
            throw;
        }
        BLSH_CUDA(cudaStreamEndCapture(w.cap, &g));
        cudaGraphExec_t ex = nullptr;
        const cudaError_t ie = cudaGraphInstantiate(&ex, g, 0);
        cudaGraphDestroy(g);
        BLSH_CUDA(ie);
        bool stale = true;   // the capture must not have grown a buffer (its key would then differ)
        QueryWork::GraphEntry chk{};
        key_of(chk);
        stale = !same(chk, e);
        if (stale) {
            cudaGraphExecDestroy(ex);
        } else {
            e.exec = ex;
            e.stats.launches = ix.stats.launches;
            if (w.graphs.size() >= 16) {
                cudaGraphExecDestroy(w.graphs.front().exec);
                w.graphs.erase(w.graphs.begin());
            }
            w.graphs.push_back(e);
        }
        ix.stats = e.stats;
    } else {
        BLSH_CUDA(cudaGraphLaunch(hit->exec, s));
        BLSH_CUDA(cudaStreamSynchronize(s));
        blsh_stats st = hit->stats;   // shape statistics of the captured call, counts of this one
        st.total_cand = w.host_scalars[0];
        st.n_items = w.host_scalars[1];
        st.union_rows = st.total_cand;
        st.pairs_scored = st.total_cand;
        if (p.hierarchy == 1 && p.min_cand == 0) st.tau = w.host_scalars[2];
        ix.stats = st;
    }
    BLSH_CUDA(cudaMemcpyAsync(out_ids, gi, (size_t)nq * k * 8, cudaMemcpyDeviceToDevice, s));
    BLSH_CUDA(cudaMemcpyAsync(out_d2, gd, (size_t)nq * k * 4, cudaMemcpyDeviceToDevice, s));
    if (out_ncand) BLSH_CUDA(cudaMemcpyAsync(out_ncand, gn, (size_t)nq * 8, cudaMemcpyDeviceToDevice, s));
    BLSH_CUDA(cudaStreamSynchronize(s));
    return true;
}

// A shard answers only the queries of its own leaves.  It routes the whole
// batch (a1; every rank must, to learn the owners), then runs a2-a5 on the compacted batch
// of its own queries -- leaf-grouped by the routing pass, so they are one contiguous run of
// lperm -- and scatters the answers back among padding rows.  The Morton hierarchy's batch
// median tau (R18) stays a statistic of the whole batch: it is taken over global_base
// before the compaction and passed on as an explicit threshold.  With keep_stages (per-query
// exports of the full batch) or for base counts, the unsharded path runs instead.
void run_query(const blsh_index& ix, const float* Q, bool q_host, int64_t nq, int k, const blsh_query_params& p,
               int64_t* out_ids, float* out_d2, unsigned long long* out_packed, int64_t* out_ncand, bool out_host,
               int64_t* out_base) {
    const bool shard = ix.leaf_lo > 0 || ix.leaf_hi < ix.G;
    if (!shard && !q_host && !out_host && !out_base && !out_packed && out_ids && out_d2 &&
        query_graph(ix, Q, nq, k, p, out_ids, out_d2, out_ncand))
        return;
    if (!shard || p.keep_stages || out_base || nq == 0) {
        run_query_core(ix, Q, q_host, nq, k, p, out_ids, out_d2, out_packed, out_ncand, out_host, out_base);
        return;
    }
    cudaStream_t s = (cudaStream_t)p.stream;
    QueryWork& w = ix.qw;
    const int ds = ix.ds, G = ix.G;
    int launches = 0;
    const bool q_direct = !q_host && ds == ix.d && (reinterpret_cast<uintptr_t>(Q) & 15u) == 0;
    const float* Qdev = Q;
    if (!q_direct) {
        w.sh_qfull.ensure((size_t)nq * ds * sizeof(float));
        if (ds != ix.d) BLSH_CUDA(cudaMemsetAsync(w.sh_qfull.p, 0, (size_t)nq * ds * sizeof(float), s));
        BLSH_CUDA(cudaMemcpy2DAsync(w.sh_qfull.p, ds * sizeof(float), Q, ix.d * sizeof(float), ix.d * sizeof(float), nq,
                                    q_host ? cudaMemcpyHostToDevice : cudaMemcpyDeviceToDevice, s));
        Qdev = w.sh_qfull.as<float>();
    }
    // carve: leaf [nq], lperm [nq], leaf counts + cursors [2G], tau, compact rows and outputs
    size_t need = 0;
    auto add = [&](size_t cnt, size_t el) { need += Arena::need(cnt, el); };
    add(nq, 4); add(nq, 4); add((size_t)2 * G, 4); add(4, 8);
    add((size_t)nq * ds, 4); add((size_t)nq * k, 8); add((size_t)nq * k, 4); add((size_t)nq * k, 8); add(nq, 8);
    add((size_t)nq * k, 8); add((size_t)nq * k, 4); add((size_t)nq * k, 8); add(nq, 8);
    w.sh_buf.ensure(need);
    Arena ar{w.sh_buf.as<char>(), 0, w.sh_buf.bytes};
    int32_t* qleaf = ar.take<int32_t>(nq);
    uint32_t* lperm = ar.take<uint32_t>(nq);
    int32_t* lcnt = ar.take<int32_t>((size_t)2 * G);
    int64_t* tau_d = ar.take<int64_t>(4);
    float* Qc = ar.take<float>((size_t)nq * ds);
    int64_t* ids_c = ar.take<int64_t>((size_t)nq * k);
    float* d2_c = ar.take<float>((size_t)nq * k);
    unsigned long long* pk_c = ar.take<unsigned long long>((size_t)nq * k);
    int64_t* nc_c = ar.take<int64_t>(nq);
    QueryArgs a{};
    a.nq = nq; a.d = ix.d; a.ds = ds; a.G = G; a.M = ix.M; a.B = ix.B; a.depth = ix.depth;
    a.quantizer = ix.quantizer; a.leaf_lo = ix.leaf_lo; a.leaf_hi = ix.leaf_hi;
    a.Q = Qdev; a.dirs = ix.dirs.as<float>(); a.mu = ix.mu.as<float>(); a.theta = ix.theta.as<float>();
    a.ntype = ix.ntype.as<int32_t>(); a.qleaf = qleaf; a.lperm = lperm; a.lcnt = lcnt;
    launches += launch_route_group(a, s);
    std::vector<int32_t> cnt_h((size_t)G);
    BLSH_CUDA(cudaMemcpyAsync(cnt_h.data(), lcnt, (size_t)G * 4, cudaMemcpyDeviceToHost, s));
    blsh_query_params p2 = p;
    p2.global_base = nullptr;
    int64_t tau = 0;
    const bool med = p.hierarchy == 1 && p.min_cand == 0;
    if (med) {   // R18 over the whole batch (check_query guarantees global_base on a shard)
        launch_median(p.global_base, nq, tau_d, s);
        ++launches;
        BLSH_CUDA(cudaMemcpyAsync(&tau, tau_d, 8, cudaMemcpyDeviceToHost, s));
    }
    BLSH_CUDA(cudaStreamSynchronize(s));
    if (med) {
        if (tau > 0) p2.min_cand = tau;
        else p2.hierarchy = 0;   // tau = 0: no query is below it, nothing widens
    }
    int64_t off = 0, nown = 0;
    for (int g = 0; g < G; ++g) {
        if (g < ix.leaf_lo) off += cnt_h[g];
        else if (g < ix.leaf_hi) nown += cnt_h[g];
    }
    const uint32_t* own = lperm + off;   // the owned queries, grouped by leaf
    launch_gather_rows(Qdev, ds, own, nown, Qc, s);
    ++launches;
    int64_t* d_ids = out_ids;
    float* d_d2 = out_d2;
    unsigned long long* d_pk = out_packed;
    int64_t* d_nc = out_ncand;
    if (out_host) {
        d_ids = out_ids ? ar.take<int64_t>((size_t)nq * k) : nullptr;
        d_d2 = out_d2 ? ar.take<float>((size_t)nq * k) : nullptr;
        d_pk = out_packed ? ar.take<unsigned long long>((size_t)nq * k) : nullptr;
        d_nc = out_ncand ? ar.take<int64_t>(nq) : nullptr;
    }
    if (nown > 0)
        run_query_core(ix, Qc, false, nown, k, p2, out_ids ? ids_c : nullptr, out_d2 ? d2_c : nullptr,
                       out_packed ? pk_c : nullptr, nc_c, false, nullptr);
    else
        ix.stats = blsh_stats{};
    launch_shard_outputs(own, nq, nown, k, ids_c, d2_c, pk_c, nc_c, d_ids, d_d2, d_pk, d_nc, s);
    launches += nown > 0 ? 2 : 1;
    if (out_host) {
        if (out_ids) BLSH_CUDA(cudaMemcpyAsync(out_ids, d_ids, (size_t)nq * k * 8, cudaMemcpyDeviceToHost, s));
        if (out_d2) BLSH_CUDA(cudaMemcpyAsync(out_d2, d_d2, (size_t)nq * k * 4, cudaMemcpyDeviceToHost, s));
        if (out_ncand) BLSH_CUDA(cudaMemcpyAsync(out_ncand, d_nc, (size_t)nq * 8, cudaMemcpyDeviceToHost, s));
        if (out_packed) BLSH_CUDA(cudaMemcpyAsync(out_packed, d_pk, (size_t)nq * k * 8, cudaMemcpyDeviceToHost, s));
    }
    BLSH_CUDA(cudaStreamSynchronize(s));
    ix.stats.nq = nq;
    ix.stats.launches += launches;
    if (med) ix.stats.tau = tau;
}

// Serving form (include/blsh.h blsh_query_pipelined): batch b is searched on p.stream from device
// staging buffer b % 2 while the copy stream uploads batch b + 1 into the other buffer and then
// downloads batch b - 1's answers.  Every batch is one run_query call on device memory, so the
// answers are those of separate blsh_query calls.  Ordering (events):
//   up[i]   on copy, after the upload of a batch into pl_q[i]    -> the search of that batch waits
//   free[i] on s,    after the search of a batch in slot i        -> the download of its answers waits
//   dl[i]   on copy, after the download of slot i's answers       -> the search two batches later waits
// The upload of batch b + 2 into slot i is queued on the copy stream after the download of batch b
// (slot i), which itself waits for free[i]: the buffer is never overwritten while in use.
void run_query_pipelined(const blsh_index& ix, int nb, const float* const* Q, int64_t nq, int k,
                         const blsh_query_params& p, int64_t* const* out_ids, float* const* out_d2,
                         int64_t* const* out_ncand) {
    cudaStream_t s = (cudaStream_t)p.stream;
    QueryWork& w = ix.qw;
    if (!w.copy) {
        BLSH_CUDA(cudaStreamCreateWithFlags(&w.copy, cudaStreamNonBlocking));
        for (int i = 0; i < 2; ++i) {
            BLSH_CUDA(cudaEventCreateWithFlags(&w.pl_up[i], cudaEventDisableTiming));
            BLSH_CUDA(cudaEventCreateWithFlags(&w.pl_free[i], cudaEventDisableTiming));
            BLSH_CUDA(cudaEventCreateWithFlags(&w.pl_dl[i], cudaEventDisableTiming));
        }
    }
    cudaStream_t cs = w.copy;
    const size_t qb = (size_t)nq * ix.d * sizeof(float);
    const size_t ib = ((size_t)nq * k * 8 + 255) & ~size_t(255);
    const size_t db = ((size_t)nq * k * 4 + 255) & ~size_t(255);
    const size_t cb = (size_t)nq * 8;
    for (int i = 0; i < 2; ++i) {
        w.pl_q[i].ensure(qb);
        w.pl_out[i].ensure(ib + db + cb);
    }
    // the copy stream starts after everything already queued on s (earlier users of the buffers)
    BLSH_CUDA(cudaEventRecord(w.pl_free[0], s));
    BLSH_CUDA(cudaStreamWaitEvent(cs, w.pl_free[0], 0));
    auto upload = [&](int b) {
        const int i = b & 1;
        BLSH_CUDA(cudaMemcpyAsync(w.pl_q[i].p, Q[b], qb, cudaMemcpyHostToDevice, cs));
        BLSH_CUDA(cudaEventRecord(w.pl_up[i], cs));
    };
    upload(0);
    int launches = 0;
    for (int b = 0; b < nb; ++b) {
        const int i = b & 1;
        if (b + 1 < nb) upload(b + 1);
        BLSH_CUDA(cudaStreamWaitEvent(s, w.pl_up[i], 0));
        if (b >= 2) BLSH_CUDA(cudaStreamWaitEvent(s, w.pl_dl[i], 0));
        char* ob = w.pl_out[i].as<char>();
        int64_t* di = reinterpret_cast<int64_t*>(ob);
        float* dd = reinterpret_cast<float*>(ob + ib);
        int64_t* dn = reinterpret_cast<int64_t*>(ob + ib + db);
        run_query(ix, w.pl_q[i].as<float>(), false, nq, k, p, di, dd, nullptr, dn, false, nullptr);
        launches += ix.stats.launches;
        BLSH_CUDA(cudaEventRecord(w.pl_free[i], s));
        BLSH_CUDA(cudaStreamWaitEvent(cs, w.pl_free[i], 0));
        BLSH_CUDA(cudaMemcpyAsync(out_ids[b], di, (size_t)nq * k * 8, cudaMemcpyDeviceToHost, cs));
        BLSH_CUDA(cudaMemcpyAsync(out_d2[b], dd, (size_t)nq * k * 4, cudaMemcpyDeviceToHost, cs));
        if (out_ncand && out_ncand[b]) BLSH_CUDA(cudaMemcpyAsync(out_ncand[b], dn, cb, cudaMemcpyDeviceToHost, cs));
        BLSH_CUDA(cudaEventRecord(w.pl_dl[i], cs));
    }
    BLSH_CUDA(cudaStreamSynchronize(cs));
    BLSH_CUDA(cudaStreamSynchronize(s));
    ix.stats.launches = launches;   // all batches' kernel launches (the other stats: the last batch)
}

static void run_query_core(const blsh_index& ix, const float* Q, bool q_host, int64_t nq, int k,
                           const blsh_query_params& p, int64_t* out_ids, float* out_d2,
                           unsigned long long* out_packed, int64_t* out_ncand, bool out_host, int64_t* out_base,
                           bool capture) {
    cudaStream_t s = (cudaStream_t)p.stream;
    if (!ix.qw.host_scalars) BLSH_CUDA(cudaMallocHost(&ix.qw.host_scalars, 4 * sizeof(int64_t)));
    QueryWork& w = ix.qw;
    const int T = p.n_probes, M = ix.M, ds = ix.ds;
    const bool keep = p.keep_stages != 0;
    const bool tm = p.timing != 0;
    blsh_stats& stt = ix.stats;
    stt = blsh_stats{};
    stt.nq = nq;
    int launches = 0;
    // ---- workspace ----
    size_t need = 0;
    auto add = [&](size_t cnt, size_t el) { need += Arena::need(cnt, el); };
    add((size_t)nq * ds, 4);            // Qd
    add(nq, 4); add((size_t)nq * M, 4); add((size_t)nq * M, 4); add(nq, 4); add(nq, 16);
    add((size_t)nq * (T + 1), 8);       // ivl
    add(nq, 8); add(nq, 8); add(nq, 4); // base cnt level
    add(nq + 1, 8); add(nq + 1, 8);     // items, item_off
    add(nq + 1, 8);                     // cand_off
    add(4, 8);                          // tau + misc
    add(nq, 4);                         // qorder
    add(nq, 4); add((size_t)2 * ix.G, 4);   // lperm, leaf counts + cursors
    if (keep) { add((size_t)nq * T, 16); add((size_t)nq * T, 4); }
    const int L = ix.L;
    for (int l = 1; l < L; ++l) {      // per-table a2-a4 stages
        add((size_t)nq * M, 4); add((size_t)nq * M, 4); add(nq, 4); add(nq, 16);
        add((size_t)nq * (T + 1), 8); add(nq, 8); add(nq, 8);
        if (keep) { add((size_t)nq * T, 16); add((size_t)nq * T, 4); }
    }
    const bool e8h = p.hierarchy == 1 && ix.quantizer == 1;   // E8 code hierarchy
    const bool list_path = L > 1 || e8h;                   // candidates as deduplicated position lists
    if (list_path) { add(nq + 1, 8); add(nq, 8); add(L, 8); add(L, 8); }
    if (e8h) { add(nq, 8); add(nq, 8); add(nq, 8); }
    if (out_host) { add((size_t)nq * k, 8); add((size_t)nq * k, 4); add(nq, 8); add((size_t)nq * k, 8); }
    w.arena.ensure(need);
    Arena ar{w.arena.as<char>(), 0, w.arena.bytes};
    w.Qd = ar.take<float>((size_t)nq * ds);
    w.qleaf = ar.take<int32_t>(nq);
    w.qt = ar.take<float>((size_t)nq * M);
    w.qcode = ar.take<int32_t>((size_t)nq * M);
    w.qoor = ar.take<int32_t>(nq);
    w.qkey = ar.take<Key128>(nq);
    w.ivl = ar.take<uint2>((size_t)nq * (T + 1));
    w.base = ar.take<int64_t>(nq);
    w.cnt = ar.take<int64_t>(nq);
    w.level = ar.take<int32_t>(nq);
    int64_t* items = ar.take<int64_t>(nq + 1);
    w.item_off = ar.take<int64_t>(nq + 1);
    int64_t* cand_off = ar.take<int64_t>(nq + 1);
    w.tau = ar.take<int64_t>(4);
    uint32_t* qorder = ar.take<uint32_t>(nq);
    uint32_t* lperm = ar.take<uint32_t>(nq);
    int32_t* lcnt = ar.take<int32_t>((size_t)2 * ix.G);
    w.pkey = keep ? ar.take<Key128>((size_t)nq * T) : nullptr;
    w.pvalid = keep ? ar.take<int32_t>((size_t)nq * T) : nullptr;
    w.tq.assign(L, QueryWork::TableQuery{});
    w.tq[0] = {w.qt, w.qcode, w.qoor, w.qkey, w.pkey, w.pvalid, w.ivl, w.base, w.cnt};
    for (int l = 1; l < L; ++l) {
        auto& t = w.tq[l];
        t.qt = ar.take<float>((size_t)nq * M);
        t.qcode = ar.take<int32_t>((size_t)nq * M);
        t.qoor = ar.take<int32_t>(nq);
        t.qkey = ar.take<Key128>(nq);
        t.ivl = ar.take<uint2>((size_t)nq * (T + 1));
        t.base = ar.take<int64_t>(nq);
        t.cnt = ar.take<int64_t>(nq);
        t.pkey = keep ? ar.take<Key128>((size_t)nq * T) : nullptr;
        t.pvalid = keep ? ar.take<int32_t>((size_t)nq * T) : nullptr;
    }
    int64_t* raw = nullptr;
    const uint2** ivl_ptrs = nullptr;
    const int64_t** cnt_ptrs = nullptr;
    if (list_path) {
        w.raw_off = ar.take<int64_t>(nq + 1);
        raw = ar.take<int64_t>(nq);
        ivl_ptrs = ar.take<const uint2*>(L);
        cnt_ptrs = ar.take<const int64_t*>(L);
    }
    int64_t *h_s = nullptr, *h_e = nullptr, *h_rows = nullptr;
    if (e8h) {
        h_s = ar.take<int64_t>(nq);
        h_e = ar.take<int64_t>(nq);
        h_rows = ar.take<int64_t>(nq);
    }
    int64_t* d_ids = out_ids;
    float* d_d2 = out_d2;
    int64_t* d_nc = out_ncand;
    unsigned long long* d_pk = out_packed;
    if (out_host) {
        int64_t* si = ar.take<int64_t>((size_t)nq * k);
        float* sd = ar.take<float>((size_t)nq * k);
        int64_t* sn = ar.take<int64_t>(nq);
        unsigned long long* sp = ar.take<unsigned long long>((size_t)nq * k);
        d_ids = out_ids ? si : nullptr;
        d_d2 = out_d2 ? sd : nullptr;
        d_nc = out_ncand ? sn : nullptr;
        d_pk = out_packed ? sp : nullptr;
    }
    w.nq = nq;
    w.T = T;
    w.k = k;
    if (tm) BLSH_CUDA(cudaEventRecord(ix.ev[0], s));
    // ---- queries into the padded layout ----
    // device queries already in the kernels' layout (d a multiple of 4, 16-byte aligned rows) are
    // read in place; otherwise they are copied (host -> device, or padded to d_stride)
    const bool q_direct = !q_host && ds == ix.d && (reinterpret_cast<uintptr_t>(Q) & 15u) == 0;
    if (!q_direct) {
        if (ds != ix.d) BLSH_CUDA(cudaMemsetAsync(w.Qd, 0, (size_t)nq * ds * sizeof(float), s));
        BLSH_CUDA(cudaMemcpy2DAsync(w.Qd, ds * sizeof(float), Q, ix.d * sizeof(float), ix.d * sizeof(float), nq,
                                    q_host ? cudaMemcpyHostToDevice : cudaMemcpyDeviceToDevice, s));
    }
    const float* Qdev = q_direct ? Q : w.Qd;
    if (tm) BLSH_CUDA(cudaEventRecord(ix.ev[1], s));
    QueryArgs a{};
    a.nq = nq; a.d = ix.d; a.ds = ds; a.G = ix.G; a.M = M; a.B = ix.B; a.depth = ix.depth;
    a.quantizer = ix.quantizer; a.leaf_lo = ix.leaf_lo; a.leaf_hi = ix.leaf_hi;
    a.probe = p.probe; a.T = T; a.hstep = p.hier_step_bits > 0 ? p.hier_step_bits : M;
    a.cperturb = p.probe == 3 ? p.curve_perturb : 0; a.msb_min = p.msb_min;
    a.rec_tau = (p.probe == 2 && p.hierarchy == 0 && p.min_cand > 0) ? p.min_cand : 0;   // R33
    a.Q = Qdev; a.dirs = ix.dirs.as<float>(); a.mu = ix.mu.as<float>(); a.theta = ix.theta.as<float>();
    a.ntype = ix.ntype.as<int32_t>(); a.A = ix.A.as<float>(); a.bvec = ix.b.as<float>(); a.Wl = ix.W.as<float>();
    a.ukey = ix.ukey.as<Key128>(); a.uoff = ix.uoff.as<uint32_t>(); a.leaf_u = ix.leaf_u.as<int64_t>();
    a.qleaf = w.qleaf; a.qt = w.qt; a.qcode = w.qcode; a.qoor = w.qoor; a.qkey = w.qkey;
    a.pkey = w.pkey; a.pvalid = w.pvalid; a.ivl = w.ivl; a.base = w.base; a.cnt = w.cnt; a.level = w.level;
    a.lperm = lperm; a.lcnt = lcnt;
    a.dr = ix.dr; a.Rh = ix.Rh.p; a.rconst = ix.rconst.as<float4>(); a.rgrp = ix.rgrp.as<uint32_t>();
    a.natom = (ix.n_owned + 7) / 8;
    a.anc = ix.anc.as<float>();
    // a1+a2
    launches += launch_route_hash(a, s);
    auto table_args = [&](int l) {   // QueryArgs of hash table l
        QueryArgs al = a;
        const auto& t = w.tq[l];
        const auto& x = *ix.xt[l - 1];
        al.A = x.A.as<float>(); al.bvec = x.b.as<float>();
        al.ukey = x.ukey.as<Key128>(); al.uoff = x.uoff.as<uint32_t>(); al.leaf_u = x.leaf_u.as<int64_t>();
        al.qt = t.qt; al.qcode = t.qcode; al.qoor = t.qoor; al.qkey = t.qkey; al.pkey = t.pkey;
        al.pvalid = t.pvalid; al.ivl = t.ivl; al.base = t.base; al.cnt = t.cnt; al.level = nullptr;
        return al;
    };
    if (L > 1) {   // tables 1..L-1: one launch
        HashTables ht{};
        ht.n = L - 1;
        for (int l = 1; l < L; ++l) {
            const QueryArgs al = table_args(l);
            ht.A[l - 1] = al.A; ht.b[l - 1] = al.bvec; ht.qt[l - 1] = al.qt; ht.qcode[l - 1] = al.qcode;
            ht.qoor[l - 1] = al.qoor; ht.qkey[l - 1] = al.qkey;
        }
        launch_hash_tables(a, ht, s);
        ++launches;
    }
    if (tm) BLSH_CUDA(cudaEventRecord(ix.ev[2], s));
    // query-tiled short-list ahead: fork the query sort + tile formation (a1/a2 outputs only)
    const int kind_pre = (list_path || out_base) ? 0 : shortlist_kind(nq, ds, ix.dr, T, k);
    if (kind_pre > 0) {
        if (!w.side) {
            BLSH_CUDA(cudaStreamCreateWithFlags(&w.side, cudaStreamNonBlocking));
            BLSH_CUDA(cudaEventCreateWithFlags(&w.ev_fork, cudaEventDisableTiming));
            BLSH_CUDA(cudaEventCreateWithFlags(&w.ev_join, cudaEventDisableTiming));
        }
        BLSH_CUDA(cudaEventRecord(w.ev_fork, s));
    }
    // a3+a4
    launch_probe_lookup(a, s); ++launches;
    for (int l = 1; l < L; ++l) { launch_probe_lookup(table_args(l), s); ++launches; }

    if (out_base) {   // blsh_query_base_counts: a1-a4 only
        BLSH_CUDA(cudaMemcpyAsync(out_base, w.base, (size_t)nq * 8, out_host ? cudaMemcpyDeviceToHost
                                                                              : cudaMemcpyDeviceToDevice, s));
        if (tm) BLSH_CUDA(cudaEventRecord(ix.ev[3], s));
        BLSH_CUDA(cudaStreamSynchronize(s));
        stt.launches = launches;
        if (tm) {
            cudaEventElapsedTime(&stt.ms_route_hash, ix.ev[1], ix.ev[2]);
            cudaEventElapsedTime(&stt.ms_probe, ix.ev[2], ix.ev[3]);
            cudaEventElapsedTime(&stt.ms_total, ix.ev[0], ix.ev[3]);
        }
        ix.has_stages = keep;
        return;
    }
    if (p.hierarchy == 2) {   // P:132 shared-MSB climb (R32): no threshold statistic
        launch_msb_climb(a, s); ++launches;
    } else if (p.hierarchy) {
        if (p.min_cand == 0) {
            launch_median(p.global_base ? p.global_base : w.base, nq, w.tau, s);
            ++launches;
        }
        if (e8h) {
            E8WidenArgs ew{};
            ew.nq = nq; ew.M = ix.M; ew.B = ix.B; ew.qleaf = w.qleaf; ew.qoor = w.qoor; ew.qcode = w.qcode; ew.base = w.base;
            ew.ukey = ix.ukey.as<Key128>(); ew.uoff = ix.uoff.as<uint32_t>(); ew.leaf_u = ix.leaf_u.as<int64_t>();
            ew.root = ix.e8_root.as<int32_t>();
            ew.lv_key = reinterpret_cast<const Key128* const*>(ix.e8_ptrs.as<char>());
            ew.lv_cum = reinterpret_cast<const int64_t* const*>(ix.e8_ptrs.as<char>() + 2 * (kE8Levels + 1) * sizeof(void*));
            ew.hlevel = w.level; ew.hs = h_s; ew.he = h_e; ew.hrows = h_rows;
            launch_e8_widen(ew, w.tau, p.min_cand, s); ++launches;
        } else {
            launch_widen(a, w.tau, p.min_cand, s); ++launches;
        }
    }
    int64_t total_raw = 0;
    if (list_path) {   // a4 across tables / with the E8 node: deduplicated union (R24, R27)
        std::vector<const uint2*> iv(L);
        std::vector<const int64_t*> cn(L);
        for (int l = 0; l < L; ++l) { iv[l] = w.tq[l].ivl; cn[l] = w.tq[l].cnt; }
        BLSH_CUDA(cudaMemcpyAsync(ivl_ptrs, iv.data(), L * sizeof(void*), cudaMemcpyHostToDevice, s));
        BLSH_CUDA(cudaMemcpyAsync(cnt_ptrs, cn.data(), L * sizeof(void*), cudaMemcpyHostToDevice, s));
        UnionArgs u{};
        u.nq = nq; u.L = L; u.T = T; u.qleaf = w.qleaf; u.qoor = w.qoor; u.ivl = ivl_ptrs; u.cnt = cnt_ptrs;
        u.pos = ix.tab_pos.as<const uint32_t*>(); u.leaf_pos = ix.leaf_pos.as<int64_t>();
        u.raw_off = w.raw_off; u.raw = raw; u.out_cnt = w.cnt;
        if (e8h) {
            u.hlevel = w.level; u.hs = h_s; u.he = h_e; u.hrows = h_rows;
            u.lv_bu = reinterpret_cast<const uint32_t* const*>(ix.e8_ptrs.as<char>() + (kE8Levels + 1) * sizeof(void*));
            u.uoff = ix.uoff.as<uint32_t>();
        }
        launch_raw_counts(u, s); ++launches;
        scan_exclusive_i64(raw, w.raw_off, nq, w.scan, s); launches += 3;
        BLSH_CUDA(cudaMemcpyAsync(&total_raw, w.raw_off + nq, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
        BLSH_CUDA(cudaStreamSynchronize(s));
        w.listbuf.ensure((size_t)std::max<int64_t>(total_raw, 1) * sizeof(uint32_t));
        u.list = w.listbuf.as<uint32_t>();
        launch_union_tables(u, ix.max_leaf_rows, s); ++launches;
    }
    w.list_valid = list_path;
    int64_t ntiles_pre = 0;
    if (kind_pre > 0) {   // side stream, overlapping a3/a4 already queued on s
        BLSH_CUDA(cudaStreamWaitEvent(w.side, w.ev_fork, 0));
        sort_queries(a, w.qsort, qorder, w.side, &launches);
        ntiles_pre = plan_tiles(a, qorder, w.tilebuf, w.scan2, w.side, &launches);
        BLSH_CUDA(cudaEventRecord(w.ev_join, w.side));
        BLSH_CUDA(cudaStreamWaitEvent(s, w.ev_join, 0));
    }
    if (tm) BLSH_CUDA(cudaEventRecord(ix.ev[3], s));
    // plan: chunking of the candidate lists
    scan_exclusive_i64(w.cnt, cand_off, nq, w.scan, s); launches += 3;
    int64_t total = 0;
    // small batches on the warp short-list plan without host round trips: chunks of 256, item
    // count and candidate total stay on the device, buffers sized by |A(q)| <= the leaf's rows
    // (R21: candidates come from the query's own leaf); one synchronisation per call
    const bool nosync = kind_pre == 0 && !list_path && nq <= small_batch_limit();
    if (!nosync) {
        BLSH_CUDA(cudaMemcpyAsync(&total, cand_off + nq, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
        BLSH_CUDA(cudaStreamSynchronize(s));
    }
    const int kind = kind_pre;   // lists: warp short-list over the positions
    const bool tiled = kind > 0;
    int64_t n_items = 0, union_rows = 0, pairs = total, kept = 0, kslots = 0;
    int screen_kind = 0;
    double qload_rows = 0.0;
    const int tcpath = kind == 2 ? 1 : 0;
    int64_t ch = 0;
    if (tiled) {
        // a5, query-tiled: sort queries by bi-level code, stream each tile's candidate union once
        int chr = 0;
        run_tiled_shortlist(a, qorder, k, w.segbuf, w.tilebuf, w.rowbuf, w.partials, w.keybuf, w.scan, d_ids, d_d2,
                            d_pk, d_nc,
                            ix.Xp.as<float>(), ix.perm.as<uint32_t>(), s, &launches, &n_items, &chr, &union_rows,
                            tm ? ix.ev[4] : nullptr, tm ? ix.ev[8] : nullptr, tm ? ix.ev[5] : nullptr, &pairs,
                            &kept, &qload_rows, kind, ntiles_pre, &kslots, &screen_kind);
        ch = chr;
        if (tm) BLSH_CUDA(cudaEventRecord(ix.ev[6], s));
    } else {
        const int64_t target = 148 * 8 * 4;
        int64_t total_cap = total;
        if (nosync) {
            // a few queries: short chunks, so that their candidates spread over many warps
            // (one warp streams its chunk with 4 rows in flight: latency-bound)
            ch = nq <= 4 ? 32 : (nq <= 32 ? 64 : 256);
            total_cap = nq * std::max<int64_t>(ix.max_leaf_rows, 1);
        } else {
            ch = (total + target - 1) / std::max<int64_t>(target, 1);
            ch = std::min<int64_t>(4096, std::max<int64_t>(256, (ch + 31) / 32 * 32));
        }
        launch_items(w.cnt, nq, (int)ch, items, s); ++launches;
        scan_exclusive_i64(items, w.item_off, nq, w.scan, s); launches += 3;
        if (nosync) {
            n_items = nq + (total_cap + ch - 1) / ch;   // >= sum of ceil(|A(q)| / ch): the grid's bound
        } else {
            BLSH_CUDA(cudaMemcpyAsync(&n_items, w.item_off + nq, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
            BLSH_CUDA(cudaStreamSynchronize(s));
        }
        const bool large_k = k > 64;
        if (large_k) w.partials.ensure((size_t)std::max<int64_t>(total_cap, 1) * sizeof(unsigned long long));
        else w.partials.ensure((size_t)std::max<int64_t>(n_items, 1) * k * sizeof(unsigned long long));
        if (tm) BLSH_CUDA(cudaEventRecord(ix.ev[4], s));
        // a5, one warp per (query, chunk)
        ShortlistArgs sa{};
        sa.nq = nq; sa.n_items = n_items; sa.d = ix.d; sa.ds = ds; sa.T = T; sa.k = k; sa.chunk = (int)ch;
        sa.Q = Qdev; sa.Xp = ix.Xp.as<float>(); sa.perm = ix.perm.as<uint32_t>(); sa.ivl = w.ivl; sa.cnt = w.cnt;
        sa.item_off = w.item_off; sa.partials = w.partials.as<unsigned long long>();
        sa.cand_off = cand_off;
        sa.list = list_path ? w.listbuf.as<uint32_t>() : nullptr;
        sa.list_off = list_path ? w.raw_off : nullptr;
        sa.cand_keys = large_k ? w.partials.as<unsigned long long>() : nullptr;
        sa.n_items_dev = nosync ? w.item_off + nq : nullptr;
        launch_shortlist(sa, s); if (n_items) ++launches;
        if (tm) BLSH_CUDA(cudaEventRecord(ix.ev[5], s));
        if (large_k) launch_select(sa.cand_keys, cand_off, nq, k, w.qoor, w.cnt, d_ids, d_d2, d_pk, d_nc, s);
        else launch_merge(sa, w.qoor, d_ids, d_d2, d_pk, d_nc, s);
        ++launches;
        if (tm) BLSH_CUDA(cudaEventRecord(ix.ev[6], s));
        union_rows = total;
    }
    if (out_host) {
        if (out_ids) BLSH_CUDA(cudaMemcpyAsync(out_ids, d_ids, (size_t)nq * k * 8, cudaMemcpyDeviceToHost, s));
        if (out_d2) BLSH_CUDA(cudaMemcpyAsync(out_d2, d_d2, (size_t)nq * k * 4, cudaMemcpyDeviceToHost, s));
        if (out_ncand) BLSH_CUDA(cudaMemcpyAsync(out_ncand, d_nc, (size_t)nq * 8, cudaMemcpyDeviceToHost, s));
        if (out_packed) BLSH_CUDA(cudaMemcpyAsync(out_packed, d_pk, (size_t)nq * k * 8, cudaMemcpyDeviceToHost, s));
    }
    if (tm) BLSH_CUDA(cudaEventRecord(ix.ev[7], s));
    if (nosync) {   // the statistics of the device-side plan
        BLSH_CUDA(cudaMemcpyAsync(&w.host_scalars[0], cand_off + nq, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
        BLSH_CUDA(cudaMemcpyAsync(&w.host_scalars[1], w.item_off + nq, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
    }
    const bool tau_dev = p.hierarchy == 1 && p.min_cand == 0;
    if (tau_dev) BLSH_CUDA(cudaMemcpyAsync(&w.host_scalars[2], w.tau, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
    if (capture) {   // query_graph: the caller launches, synchronises and reads host_scalars
        stt.launches = launches;
        stt.chunk = (int32_t)ch;
        return;
    }
    BLSH_CUDA(cudaStreamSynchronize(s));
    if (nosync) {
        total = w.host_scalars[0];
        n_items = w.host_scalars[1];
        union_rows = total;
        pairs = total;
    }
    stt.total_cand = total;
    stt.n_items = n_items;
    stt.chunk = (int32_t)ch;
    stt.launches = launches;
    stt.shortlist_bytes = (double)total * ix.d * 4.0 + (double)total * 4.0 +
                          (k > 64 && !tiled ? (double)total * 8.0 : (double)n_items * k * 8.0);
    stt.tiled = tiled ? (tcpath ? 2 : 1) : 0;
    stt.union_rows = union_rows;
    stt.pairs_kept = kept;
    // bytes the streaming kernel reads per union row: fp16 screen: the fp16 row (2 dr), its (row, mask, K slot)
    // entry and its bound constants (16 + 16); TF32 screen / SIMT tiled: the fp32 row + its entry
    const int row_bytes = screen_kind == 1 ? 2 * ix.dr + 32 : 4 * ds + (screen_kind == 2 ? 16 : 8);
    stt.k_slots = kslots;
    stt.screen_kind = screen_kind;
    stt.screen_row_bytes = tiled ? row_bytes : 4 * ix.d + 4;
    stt.union_bytes = tiled ? (double)union_rows * row_bytes + qload_rows * 4.0 * ds + (double)kslots * 32.0 * 4.0
                            : stt.shortlist_bytes;
    stt.pairs_scored = pairs;
    stt.shortlist_flops = 3.0 * ix.d * (double)total;
    if (p.hierarchy == 1) {
        int64_t tau = p.min_cand;
        if (tau_dev) tau = w.host_scalars[2];
        stt.tau = tau;
    }
    if (tm) {
        cudaEventElapsedTime(&stt.ms_route_hash, ix.ev[1], ix.ev[2]);
        cudaEventElapsedTime(&stt.ms_probe, ix.ev[2], ix.ev[3]);
        cudaEventElapsedTime(&stt.ms_plan, ix.ev[3], ix.ev[4]);
        cudaEventElapsedTime(&stt.ms_shortlist, ix.ev[4], ix.ev[5]);
        if (tiled) {
            cudaEventElapsedTime(&stt.ms_screen, ix.ev[4], ix.ev[8]);
            cudaEventElapsedTime(&stt.ms_rescore, ix.ev[8], ix.ev[5]);
        } else {
            stt.ms_screen = stt.ms_shortlist;
        }
        cudaEventElapsedTime(&stt.ms_merge, ix.ev[5], ix.ev[6]);
        cudaEventElapsedTime(&stt.ms_total, ix.ev[0], ix.ev[7]);
    }
    ix.has_stages = keep;
}

}  // namespace blsh

namespace {

blsh_status check_query(const blsh_index* idx, const float* Q, int64_t nq, int32_t k, const blsh_query_params* p) {
    if (!idx) return fail(BLSH_ERR_INVALID, "index is NULL");
    if (!p) return fail(BLSH_ERR_INVALID, "params is NULL");
    if (nq < 0 || nq >= (int64_t(1) << 31)) return fail(BLSH_ERR_INVALID, "nq must be in [0, 2^31)");
    if (nq > 0 && !Q) return fail(BLSH_ERR_INVALID, "Q is NULL");
    if (k < 1) return fail(BLSH_ERR_INVALID, "k must be >= 1");
    if (k > 1024) return fail(BLSH_ERR_UNSUPPORTED, "k > 1024");
    if (p->n_probes < 1) return fail(BLSH_ERR_INVALID, "n_probes must be >= 1");
    if (p->probe == 0 && p->n_probes != 1) return fail(BLSH_ERR_INVALID, "standard probing uses n_probes = 1");
    if (p->probe == 1) {
        if (idx->quantizer != 0) return fail(BLSH_ERR_INVALID, "multiprobe needs a Z^M index");
        if (idx->M > 10) return fail(BLSH_ERR_UNSUPPORTED, "multiprobe needs M <= 10");
        if (p->n_probes > ipow3(idx->M)) return fail(BLSH_ERR_INVALID, "n_probes > 3^M");
    } else if (p->probe == 2) {
        if (idx->quantizer != 1) return fail(BLSH_ERR_INVALID, "lattice probing needs an E8 index");
        if (p->n_probes > 256) return fail(BLSH_ERR_INVALID, "n_probes > 256");
    } else if (p->probe == 3) {
        if (idx->quantizer != 0) return fail(BLSH_ERR_INVALID, "Morton-curve probing needs a Z^M index");
    } else if (p->probe != 0) {
        return fail(BLSH_ERR_INVALID, "probe must be 0, 1, 2 or 3");
    }
    if (p->n_probes > 256) return fail(BLSH_ERR_UNSUPPORTED, "n_probes > 256");
    if (p->curve_perturb < 0 || p->curve_perturb > idx->M)
        return fail(BLSH_ERR_INVALID, "curve_perturb must be in [0, M]");
    if (p->curve_perturb > 0 && p->probe != 3) return fail(BLSH_ERR_INVALID, "curve_perturb needs probe = 3");
    if (p->hierarchy < 0 || p->hierarchy > 2) return fail(BLSH_ERR_INVALID, "hierarchy must be 0, 1 or 2");
    if (p->hierarchy == 2 && idx->quantizer != 0) return fail(BLSH_ERR_INVALID, "the shared-MSB climb needs a Z^M index");
    if (p->msb_min < 0 || p->msb_min > idx->B * idx->M) return fail(BLSH_ERR_INVALID, "msb_min must be in [0, B*M]");
    if (p->hierarchy == 2) {
        if (idx->L > 1) return fail(BLSH_ERR_UNSUPPORTED, "the Morton hierarchy is defined for one table (R24)");
    } else if (p->hierarchy) {
        if (idx->L > 1) return fail(BLSH_ERR_UNSUPPORTED, "the Morton hierarchy is defined for one table (R24)");
        if (p->hier_step_bits < 0 || p->hier_step_bits > idx->M) return fail(BLSH_ERR_INVALID, "hier_step_bits must be in [0, M]");
        if (p->min_cand < 0) return fail(BLSH_ERR_INVALID, "min_cand must be >= 0");
        if (p->min_cand == 0 && idx->world > 1 && !p->global_base)
            return fail(BLSH_ERR_INVALID, "batch-median tau on a sharded index needs p->global_base "
                                          "(blsh_query_base_counts summed over ranks) or an explicit min_cand");
    }
    if (p->min_cand < 0) return fail(BLSH_ERR_INVALID, "min_cand must be >= 0");
    if (p->probe == 2 && p->hierarchy == 0 && p->min_cand > 0 && idx->L > 1)
        return fail(BLSH_ERR_UNSUPPORTED, "recursive lattice probing (min_cand without hierarchy, R33) needs L = 1");
    if (p->global_base && !is_device_ptr(p->global_base)) return fail(BLSH_ERR_INVALID, "global_base must be device memory");
    return BLSH_OK;
}

}  // namespace

extern "C" {

blsh_status blsh_query(const blsh_index* idx, const float* Q, int64_t nq, int32_t k, const blsh_query_params* p,
                       int64_t* out_ids, float* out_dist2, int64_t* out_ncand) {
    blsh_status c = check_query(idx, Q, nq, k, p);
    if (c != BLSH_OK) return c;
    if (nq > 0 && (!out_ids || !out_dist2)) return fail(BLSH_ERR_INVALID, "outputs are NULL");
    if (nq == 0) return BLSH_OK;
    const bool q_host = !is_device_ptr(Q);
    const bool o_host = !is_device_ptr(out_ids);
    if (o_host != !is_device_ptr(out_dist2) || (out_ncand && o_host != !is_device_ptr(out_ncand)))
        return fail(BLSH_ERR_INVALID, "outputs must all be host or all be device memory");
    return guarded([&] { blsh::run_query(*idx, Q, q_host, nq, k, *p, out_ids, out_dist2, nullptr, out_ncand, o_host, nullptr); });
}

blsh_status blsh_query_pipelined(const blsh_index* idx, int32_t n_batches, const float* const* Q, int64_t nq, int32_t k,
                                 const blsh_query_params* p, int64_t* const* out_ids, float* const* out_dist2,
                                 int64_t* const* out_ncand) {
    if (n_batches < 0) return fail(BLSH_ERR_INVALID, "n_batches must be >= 0");
    if (n_batches == 0) return BLSH_OK;
    if (!Q || !out_ids || !out_dist2) return fail(BLSH_ERR_INVALID, "pointer arrays are NULL");
    for (int32_t b = 0; b < n_batches; ++b) {
        blsh_status c = check_query(idx, Q[b], nq, k, p);
        if (c != BLSH_OK) return c;
        if (nq == 0) continue;
        if (!out_ids[b] || !out_dist2[b]) return fail(BLSH_ERR_INVALID, "outputs are NULL");
        if (is_device_ptr(Q[b]) || is_device_ptr(out_ids[b]) || is_device_ptr(out_dist2[b]) ||
            (out_ncand && out_ncand[b] && is_device_ptr(out_ncand[b])))
            return fail(BLSH_ERR_INVALID, "blsh_query_pipelined takes host buffers only");
    }
    if (nq == 0) return BLSH_OK;
    return guarded([&] { blsh::run_query_pipelined(*idx, n_batches, Q, nq, k, *p, out_ids, out_dist2, out_ncand); });
}

blsh_status blsh_query_packed(const blsh_index* idx, const float* Q, int64_t nq, int32_t k, const blsh_query_params* p,
                              uint64_t* out_packed, int64_t* out_ncand) {
    blsh_status c = check_query(idx, Q, nq, k, p);
    if (c != BLSH_OK) return c;
    if (nq > 0 && !out_packed) return fail(BLSH_ERR_INVALID, "out_packed is NULL");
    if (idx->n >= (int64_t(1) << 32)) return fail(BLSH_ERR_UNSUPPORTED, "packed lists need n < 2^32");
    if (nq == 0) return BLSH_OK;
    const bool q_host = !is_device_ptr(Q);
    const bool o_host = !is_device_ptr(out_packed);
    if (out_ncand && o_host != !is_device_ptr(out_ncand))
        return fail(BLSH_ERR_INVALID, "outputs must all be host or all be device memory");
    return guarded([&] {
        blsh::run_query(*idx, Q, q_host, nq, k, *p, nullptr, nullptr, reinterpret_cast<unsigned long long*>(out_packed),
                        out_ncand, o_host, nullptr);
    });
}

blsh_status blsh_query_base_counts(const blsh_index* idx, const float* Q, int64_t nq, const blsh_query_params* p,
                                   int64_t* out_base) {
    if (!p) return fail(BLSH_ERR_INVALID, "params is NULL");
    blsh_query_params p2 = *p;
    p2.hierarchy = 0;     // the base set only: widening is not part of A0
    p2.global_base = nullptr;
    blsh_status c = check_query(idx, Q, nq, 1, &p2);
    if (c != BLSH_OK) return c;
    if (idx->L > 1) return fail(BLSH_ERR_UNSUPPORTED, "base counts serve the hierarchy, which needs L = 1");
    if (nq > 0 && !out_base) return fail(BLSH_ERR_INVALID, "out_base is NULL");
    if (nq == 0) return BLSH_OK;
    const bool q_host = !is_device_ptr(Q);
    const bool o_host = !is_device_ptr(out_base);
    return guarded([&] {
        blsh::run_query(*idx, Q, q_host, nq, 1, p2, nullptr, nullptr, nullptr, nullptr, o_host, out_base);
    });
}

blsh_status blsh_merge_topk(const uint64_t* packed, int32_t n_lists, int64_t nq, int32_t k, int64_t* out_ids,
                            float* out_dist2, void* stream) {
    if (n_lists < 1 || nq < 0 || k < 1) return fail(BLSH_ERR_INVALID, "bad sizes");
    if (k > 1024) return fail(BLSH_ERR_UNSUPPORTED, "k > 1024");
    if (nq == 0) return BLSH_OK;
    if (!packed || !out_ids || !out_dist2) return fail(BLSH_ERR_INVALID, "NULL pointer");
    if (!is_device_ptr(packed)) return fail(BLSH_ERR_INVALID, "packed must be device memory");
    const bool o_host = !is_device_ptr(out_ids);
    cudaStream_t s = (cudaStream_t)stream;
    return guarded([&] {
        blsh::DevBuf si, sd;
        int64_t* di = out_ids;
        float* dd = out_dist2;
        if (o_host) {
            si.alloc((size_t)nq * k * 8);
            sd.alloc((size_t)nq * k * 4);
            di = si.as<int64_t>();
            dd = sd.as<float>();
        }
        blsh::merge_lists(reinterpret_cast<const unsigned long long*>(packed), n_lists, nq, k, di, dd, s);
        if (o_host) {
            BLSH_CUDA(cudaMemcpyAsync(out_ids, di, (size_t)nq * k * 8, cudaMemcpyDeviceToHost, s));
            BLSH_CUDA(cudaMemcpyAsync(out_dist2, dd, (size_t)nq * k * 4, cudaMemcpyDeviceToHost, s));
        }
        BLSH_CUDA(cudaStreamSynchronize(s));
    });
}

blsh_status blsh_index_info(const blsh_index* idx, blsh_info* out) {
    if (!idx || !out) return fail(BLSH_ERR_INVALID, "NULL pointer");
    out->n = idx->n;
    out->n_owned = idx->n_owned;
    out->nu = idx->nu;
    out->d = idx->d;
    out->d_stride = idx->ds;
    out->G = idx->G;
    out->M = idx->M;
    out->B = idx->B;
    out->quantizer = idx->quantizer;
    out->leaf_lo = idx->leaf_lo;
    out->leaf_hi = idx->leaf_hi;
    out->device_bytes = (int64_t)(idx->A.bytes + idx->b.bytes + idx->W.bytes + idx->dirs.bytes + idx->mu.bytes +
                                  idx->theta.bytes + idx->ntype.bytes + idx->Xp.bytes + idx->perm.bytes +
                                  idx->ukey.bytes + idx->uleaf.bytes + idx->uoff.bytes + idx->leaf_u.bytes +
                                  idx->pt_leaf.bytes + idx->pt_code.bytes + idx->pt_key.bytes);
    out->build_ms = idx->build_ms;
    out->n_tables = idx->L;
    out->pad_ = 0;
    for (const auto& t : idx->xt)
        out->device_bytes += (int64_t)(t->A.bytes + t->b.bytes + t->ukey.bytes + t->uleaf.bytes + t->uoff.bytes +
                                       t->leaf_u.bytes + t->pos.bytes + t->perm.bytes);
    return BLSH_OK;
}

blsh_status blsh_last_stats(const blsh_index* idx, blsh_stats* out) {
    if (!idx || !out) return fail(BLSH_ERR_INVALID, "NULL pointer");
    *out = idx->stats;
    return BLSH_OK;
}

blsh_status blsh_export(const blsh_index* idx, int32_t what, void* dst, size_t cap, size_t* needed) {
    if (!idx) return fail(BLSH_ERR_INVALID, "index is NULL");
    const int table = what >> 8;   // BLSH_EX_TABLE(l, item): table l of an L-table index
    what &= 0xFF;
    if (table < 0 || table >= idx->L) return fail(BLSH_ERR_INVALID, "table out of range");
    const blsh::ExtraTable* xt = table > 0 ? idx->xt[table - 1].get() : nullptr;
    if (xt && !(what == BLSH_EX_A || what == BLSH_EX_B || what == BLSH_EX_PERM || what == BLSH_EX_UKEY ||
                what == BLSH_EX_ULEAF || what == BLSH_EX_UOFF || what == BLSH_EX_LEAF_U ||
                (what >= BLSH_EX_Q_T && what <= BLSH_EX_Q_INTERVALS && what != BLSH_EX_Q_LEVEL &&
                 what != BLSH_EX_Q_TAU && what != BLSH_EX_Q_LEAF)))
        return fail(BLSH_ERR_INVALID, "item is not per table");
    const std::vector<float>& A_h = xt ? xt->A_h : idx->A_h;
    const std::vector<float>& b_h = xt ? xt->b_h : idx->b_h;
    const void* perm_p = xt ? xt->perm.p : idx->perm.p;
    const void* ukey_p = xt ? xt->ukey.p : idx->ukey.p;
    const void* uleaf_p = xt ? xt->uleaf.p : idx->uleaf.p;
    const void* uoff_p = xt ? xt->uoff.p : idx->uoff.p;
    const int64_t nu = xt ? xt->nu : idx->nu;
    const std::vector<int64_t>& leaf_u_h = xt ? xt->leaf_u_h : idx->leaf_u_h;
    const int64_t G = idx->G, M = idx->M, d = idx->d, nn = G > 1 ? G - 1 : 0;
    const blsh::QueryWork& w = idx->qw;
    blsh::QueryWork::TableQuery tq0{w.qt, w.qcode, w.qoor, w.qkey, w.pkey, w.pvalid, w.ivl, w.base, w.cnt};
    const blsh::QueryWork::TableQuery tq = (table > 0 && (size_t)table < w.tq.size()) ? w.tq[table] : tq0;
    if (table > 0 && (size_t)table >= w.tq.size() && what >= BLSH_EX_Q_T)
        return fail(BLSH_ERR_INVALID, "last query without keep_stages");
    const int64_t nq = w.nq;
    const int T = w.T;
    const void* host_src = nullptr;
    const void* dev_src = nullptr;
    size_t bytes = 0;
    std::vector<char> tmp;
    auto need_q = [&]() -> bool { return idx->has_stages; };
    auto need_pt = [&]() -> bool { return idx->has_pt; };
    switch (what) {
        case BLSH_EX_A: host_src = A_h.data(); bytes = A_h.size() * 4; break;
        case BLSH_EX_B: host_src = b_h.data(); bytes = b_h.size() * 4; break;
        case BLSH_EX_W: host_src = idx->W_h.data(); bytes = idx->W_h.size() * 4; break;
        case BLSH_EX_DIRS: host_src = idx->dirs_h.data(); bytes = (size_t)nn * d * 4; break;
        case BLSH_EX_MU: host_src = idx->mu_h.data(); bytes = (size_t)nn * d * 4; break;
        case BLSH_EX_THETA: host_src = idx->theta_h.data(); bytes = (size_t)nn * 4; break;
        case BLSH_EX_NTYPE: host_src = idx->ntype_h.data(); bytes = (size_t)nn * 4; break;
        case BLSH_EX_DIAM2: host_src = idx->diam2_h.data(); bytes = (size_t)nn * 8; break;
        case BLSH_EX_DA2: host_src = idx->da2_h.data(); bytes = (size_t)nn * 8; break;
        case BLSH_EX_PERM: {
            bytes = (size_t)idx->n_owned * 8;
            if (dst && cap >= bytes && bytes) {
                std::vector<uint32_t> p32(idx->n_owned);
                if (cudaMemcpy(p32.data(), perm_p, p32.size() * 4, cudaMemcpyDeviceToHost) != cudaSuccess)
                    return fail(BLSH_ERR_CUDA, "export copy failed");
                int64_t* o = (int64_t*)dst;
                for (size_t i = 0; i < p32.size(); ++i) o[i] = p32[i];
            }
            if (needed) *needed = bytes;
            return (dst && cap >= bytes) ? BLSH_OK : fail(BLSH_ERR_INVALID, "dst too small");
        }
        case BLSH_EX_UKEY: {
            bytes = (size_t)nu * 16;
            if (dst && cap >= bytes && bytes) {
                std::vector<blsh::Key128> k(nu);
                if (cudaMemcpy(k.data(), ukey_p, k.size() * 16, cudaMemcpyDeviceToHost) != cudaSuccess)
                    return fail(BLSH_ERR_CUDA, "export copy failed");
                uint64_t* o = (uint64_t*)dst;
                for (size_t i = 0; i < k.size(); ++i) { o[2 * i] = k[i].hi; o[2 * i + 1] = k[i].lo; }
            }
            if (needed) *needed = bytes;
            return (dst && cap >= bytes) ? BLSH_OK : fail(BLSH_ERR_INVALID, "dst too small");
        }
        case BLSH_EX_ULEAF: dev_src = uleaf_p; bytes = (size_t)nu * 4; break;
        case BLSH_EX_RGRP: dev_src = idx->rgrp.p; bytes = (size_t)idx->n_owned * 4; break;
        case BLSH_EX_GSTART: dev_src = idx->gstart.p; bytes = (size_t)(idx->nanchor + 1) * 8; break;
        case BLSH_EX_UOFF: {
            bytes = (size_t)(nu + 1) * 8;
            if (dst && cap >= bytes) {
                std::vector<uint32_t> u(nu + 1);
                if (cudaMemcpy(u.data(), uoff_p, u.size() * 4, cudaMemcpyDeviceToHost) != cudaSuccess)
                    return fail(BLSH_ERR_CUDA, "export copy failed");
                int64_t* o = (int64_t*)dst;
                for (size_t i = 0; i < u.size(); ++i) o[i] = u[i];
            }
            if (needed) *needed = bytes;
            return (dst && cap >= bytes) ? BLSH_OK : fail(BLSH_ERR_INVALID, "dst too small");
        }
        case BLSH_EX_LEAF_U: host_src = leaf_u_h.data(); bytes = (size_t)(G + 1) * 8; break;
        case BLSH_EX_POINT_LEAF:
            if (!need_pt()) return fail(BLSH_ERR_INVALID, "build without keep_stages");
            dev_src = idx->pt_leaf.p; bytes = (size_t)idx->n * 4; break;
        case BLSH_EX_POINT_CODE:
            if (!need_pt()) return fail(BLSH_ERR_INVALID, "build without keep_stages");
            dev_src = idx->pt_code.p; bytes = (size_t)idx->n * M * 4; break;
        case BLSH_EX_POINT_KEY: {
            if (!need_pt()) return fail(BLSH_ERR_INVALID, "build without keep_stages");
            bytes = (size_t)idx->n * 16;
            if (dst && cap >= bytes && bytes) {
                std::vector<blsh::Key128> k(idx->n);
                if (cudaMemcpy(k.data(), idx->pt_key.p, k.size() * 16, cudaMemcpyDeviceToHost) != cudaSuccess)
                    return fail(BLSH_ERR_CUDA, "export copy failed");
                uint64_t* o = (uint64_t*)dst;
                for (size_t i = 0; i < k.size(); ++i) { o[2 * i] = k[i].hi; o[2 * i + 1] = k[i].lo; }
            }
            if (needed) *needed = bytes;
            return (dst && cap >= bytes) ? BLSH_OK : fail(BLSH_ERR_INVALID, "dst too small");
        }
        default: break;
    }
    if (what == BLSH_EX_Q_CAND_OFF || what == BLSH_EX_Q_CAND) {
        if (!need_q() || !w.list_valid) return fail(BLSH_ERR_INVALID, "last query without keep_stages or without lists");
        std::vector<int64_t> roff(nq + 1), cnt(nq);
        if (cudaMemcpy(roff.data(), w.raw_off, (nq + 1) * 8, cudaMemcpyDeviceToHost) != cudaSuccess ||
            cudaMemcpy(cnt.data(), w.cnt, nq * 8, cudaMemcpyDeviceToHost) != cudaSuccess)
            return fail(BLSH_ERR_CUDA, "export copy failed");
        int64_t tot = 0;
        for (int64_t q = 0; q < nq; ++q) tot += cnt[q];
        bytes = what == BLSH_EX_Q_CAND_OFF ? (size_t)(nq + 1) * 8 : (size_t)tot * 8;
        if (needed) *needed = bytes;
        if (!dst || cap < bytes) return fail(BLSH_ERR_INVALID, "dst too small");
        int64_t* o = (int64_t*)dst;
        if (what == BLSH_EX_Q_CAND_OFF) {
            o[0] = 0;
            for (int64_t q = 0; q < nq; ++q) o[q + 1] = o[q] + cnt[q];
            return BLSH_OK;
        }
        std::vector<uint32_t> lst((size_t)std::max<int64_t>(roff[nq], 1)), p32((size_t)std::max<int64_t>(idx->n_owned, 1));
        if (cudaMemcpy(lst.data(), w.listbuf.p, (size_t)roff[nq] * 4, cudaMemcpyDeviceToHost) != cudaSuccess ||
            cudaMemcpy(p32.data(), idx->perm.p, (size_t)idx->n_owned * 4, cudaMemcpyDeviceToHost) != cudaSuccess)
            return fail(BLSH_ERR_CUDA, "export copy failed");
        int64_t k = 0;
        for (int64_t q = 0; q < nq; ++q) {
            const int64_t s0 = k;
            for (int64_t i = 0; i < cnt[q]; ++i) o[k++] = p32[lst[roff[q] + i]];
            std::sort(o + s0, o + k);
        }
        return BLSH_OK;
    }
    if (what >= BLSH_EX_Q_LEAF && what <= BLSH_EX_Q_INTERVALS) {
        if (!need_q()) return fail(BLSH_ERR_INVALID, "last query without keep_stages");
        switch (what) {
            case BLSH_EX_Q_LEAF: dev_src = w.qleaf; bytes = (size_t)nq * 4; break;
            case BLSH_EX_Q_T: dev_src = tq.qt; bytes = (size_t)nq * M * 4; break;
            case BLSH_EX_Q_CODE: dev_src = tq.qcode; bytes = (size_t)nq * M * 4; break;
            case BLSH_EX_Q_OOR: {
                bytes = (size_t)nq * 4;
                if (dst && cap >= bytes) {
                    if (cudaMemcpy(dst, tq.qoor, bytes, cudaMemcpyDeviceToHost) != cudaSuccess)
                        return fail(BLSH_ERR_CUDA, "export copy failed");
                    int32_t* o = (int32_t*)dst;
                    for (int64_t i = 0; i < nq; ++i) o[i] &= ~2;   // hide the shard bit (1 range, 4 non-finite)
                }
                if (needed) *needed = bytes;
                return (dst && cap >= bytes) ? BLSH_OK : fail(BLSH_ERR_INVALID, "dst too small");
            }
            case BLSH_EX_Q_KEY:
            case BLSH_EX_Q_PKEY: {
                const int64_t cnt = what == BLSH_EX_Q_KEY ? nq : nq * T;
                bytes = (size_t)cnt * 16;
                if (dst && cap >= bytes && bytes) {
                    std::vector<blsh::Key128> k(cnt);
                    std::vector<int32_t> oor(nq);
                    if (cudaMemcpy(k.data(), what == BLSH_EX_Q_KEY ? (void*)tq.qkey : (void*)tq.pkey, bytes,
                                   cudaMemcpyDeviceToHost) != cudaSuccess ||
                        cudaMemcpy(oor.data(), tq.qoor, nq * 4, cudaMemcpyDeviceToHost) != cudaSuccess)
                        return fail(BLSH_ERR_CUDA, "export copy failed");
                    uint64_t* o = (uint64_t*)dst;
                    for (int64_t i = 0; i < cnt; ++i) {
                        const bool zero = what == BLSH_EX_Q_KEY && (oor[i] & 1);
                        o[2 * i] = zero ? 0 : k[i].hi;
                        o[2 * i + 1] = zero ? 0 : k[i].lo;
                    }
                }
                if (needed) *needed = bytes;
                return (dst && cap >= bytes) ? BLSH_OK : fail(BLSH_ERR_INVALID, "dst too small");
            }
            case BLSH_EX_Q_PVALID: dev_src = tq.pvalid; bytes = (size_t)nq * T * 4; break;
            case BLSH_EX_Q_BASE: dev_src = tq.base; bytes = (size_t)nq * 8; break;
            case BLSH_EX_Q_LEVEL: dev_src = w.level; bytes = (size_t)nq * 4; break;
            case BLSH_EX_Q_TAU: host_src = &idx->stats.tau; bytes = 8; break;
            case BLSH_EX_Q_INTERVALS: {
                bytes = (size_t)nq * (T + 1) * 16;
                if (dst && cap >= bytes && bytes) {
                    std::vector<uint2> iv((size_t)nq * (T + 1));
                    if (cudaMemcpy(iv.data(), tq.ivl, iv.size() * 8, cudaMemcpyDeviceToHost) != cudaSuccess)
                        return fail(BLSH_ERR_CUDA, "export copy failed");
                    int64_t* o = (int64_t*)dst;
                    for (size_t i = 0; i < iv.size(); ++i) { o[2 * i] = iv[i].x; o[2 * i + 1] = iv[i].y; }
                }
                if (needed) *needed = bytes;
                return (dst && cap >= bytes) ? BLSH_OK : fail(BLSH_ERR_INVALID, "dst too small");
            }
            default: break;
        }
    }
    if (!host_src && !dev_src && bytes == 0 && what != BLSH_EX_Q_TAU) {
        if (needed) *needed = 0;
        switch (what) {
            case BLSH_EX_A: case BLSH_EX_B: case BLSH_EX_W: case BLSH_EX_DIRS: case BLSH_EX_MU: case BLSH_EX_THETA:
            case BLSH_EX_NTYPE: case BLSH_EX_DIAM2: case BLSH_EX_DA2: case BLSH_EX_ULEAF: case BLSH_EX_LEAF_U:
            case BLSH_EX_Q_LEAF: case BLSH_EX_Q_T: case BLSH_EX_Q_CODE: case BLSH_EX_Q_PVALID: case BLSH_EX_Q_BASE:
            case BLSH_EX_Q_LEVEL: case BLSH_EX_POINT_LEAF: case BLSH_EX_POINT_CODE:
                return BLSH_OK;
            default:
                return fail(BLSH_ERR_INVALID, "unknown export item");
        }
    }
    if (needed) *needed = bytes;
    if (!dst || cap < bytes) return fail(BLSH_ERR_INVALID, "dst too small");
    if (bytes == 0) return BLSH_OK;
    if (host_src) {
        std::memcpy(dst, host_src, bytes);
        return BLSH_OK;
    }
    if (cudaMemcpy(dst, dev_src, bytes, cudaMemcpyDeviceToHost) != cudaSuccess)
        return fail(BLSH_ERR_CUDA, "export copy failed");
    return BLSH_OK;
}

}  // extern "C"
