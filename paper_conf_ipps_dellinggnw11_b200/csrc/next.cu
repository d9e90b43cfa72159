// next.cu -- SURVEY.md §8(f) rows built on top of finished trees (never on the
// hot path of a3):
//   NEXT-1 parent pointers (§VII-A "we check whether the identity d(v) =
//          d(u) + l(u,v) holds"), in the ORIGINAL graph (reading R14);
//   NEXT-3 exact betweenness and reach (§VII-B), readings R16/R17.
#include <algorithm>

#include "device.cuh"
#include "kernels.h"

namespace phast {
namespace {
constexpr int SWEEP_THREADS = 256;
// ------------------------------------------------------------------ NEXT-1 parent pointers
// After a sweep every label is final, so the parent pass has no dependencies: one
// grid-stride pass over (vertex, 16-byte lane) items.  Each lane owns W trees of the
// row; it scans v's original in-arcs in input order and keeps, per tree, the tail of
// the first tight arc (§VII-A).  The identity is tested as d(u) <= d(v)
// and d(v) - d(u) = l, which equals d(u) + l = d(v) exactly (no 32-bit overflow).
// The scan stops once every finite tree of the lane has its parent.
// PLUS (hierarchy parents, reading R19): a second in-arc CSR (A-up in-arcs) is scanned
// after the first (A-down in-arcs) for the trees still without a parent.
template <int K, bool PLUS>
__global__ void __launch_bounds__(SWEEP_THREADS) parents_kernel(const uint32_t* __restrict__ in_first,
                                                                const uint2* __restrict__ in_arc,
                                                                const uint32_t* __restrict__ in_first2,
                                                                const uint2* __restrict__ in_arc2,
                                                                const uint32_t* __restrict__ d,
                                                                uint32_t* __restrict__ parent, uint32_t n,
                                                                Sources src) {
    constexpr uint32_t W = RowT<K>::W;
    constexpr uint32_t G = K / W;
    using T = typename RowT<K>::T;
    const uint64_t total = (uint64_t)n * G;
    for (uint64_t t = (uint64_t)blockIdx.x * SWEEP_THREADS + threadIdx.x; t < total;
         t += (uint64_t)gridDim.x * SWEEP_THREADS) {
        const uint32_t v = (uint32_t)(t / G), lane = (uint32_t)(t % G);
        const T rv = __ldg(reinterpret_cast<const T*>(d + (size_t)v * K) + lane);
        const uint32_t* dv = reinterpret_cast<const uint32_t*>(&rv);
        uint32_t p[W];
        uint32_t need = 0;
#pragma unroll
        for (uint32_t q = 0; q < W; q++) {
            p[q] = INF;
            if (dv[q] != INF) need |= 1u << q;
        }
        for (int pass = 0; pass < (PLUS ? 2 : 1); pass++) {
            const uint32_t* f = pass ? in_first2 : in_first;
            const uint2* arcs = pass ? in_arc2 : in_arc;
            const uint32_t e1 = __ldg(&f[v + 1]);
            for (uint32_t e = __ldg(&f[v]); need && e < e1; e++) {
                const uint2 a = __ldg(&arcs[e]);
                const T ru = __ldg(reinterpret_cast<const T*>(d + (size_t)a.x * K) + lane);
                const uint32_t* du = reinterpret_cast<const uint32_t*>(&ru);
#pragma unroll
                for (uint32_t q = 0; q < W; q++)
                    if (((need >> q) & 1u) && du[q] <= dv[q] && dv[q] - du[q] == a.y) {
                        p[q] = a.x;
                        need &= ~(1u << q);
                    }
            }
        }
#pragma unroll
        for (uint32_t q = 0; q < W; q++)
            if (src.s[lane * W + q] == v) p[q] = v;   // the root of tree lane*W+q
        T out;
        uint32_t* po = reinterpret_cast<uint32_t*>(&out);
#pragma unroll
        for (uint32_t q = 0; q < W; q++) po[q] = p[q];
        reinterpret_cast<T*>(parent + (size_t)v * K)[lane] = out;
    }
}

// any k (the caller's row width is not one of the vector widths): one thread per
// (vertex, tree) item, same scan and tie rule
__global__ void __launch_bounds__(SWEEP_THREADS) parents_any_kernel(const uint32_t* __restrict__ in_first,
                                                                    const uint2* __restrict__ in_arc,
                                                                    const uint32_t* __restrict__ d,
                                                                    uint32_t* __restrict__ parent, uint32_t n,
                                                                    uint32_t k, Sources src) {
    const uint64_t total = (uint64_t)n * k;
    for (uint64_t t = (uint64_t)blockIdx.x * SWEEP_THREADS + threadIdx.x; t < total;
         t += (uint64_t)gridDim.x * SWEEP_THREADS) {
        const uint32_t v = (uint32_t)(t / k), i = (uint32_t)(t % k);
        const uint32_t dv = __ldg(&d[t]);
        uint32_t p = INF;
        if (dv != INF) {
            const uint32_t e1 = __ldg(&in_first[v + 1]);
            for (uint32_t e = __ldg(&in_first[v]); e < e1; e++) {
                const uint2 a = __ldg(&in_arc[e]);
                const uint32_t du = __ldg(&d[(size_t)a.x * k + i]);
                if (du <= dv && dv - du == a.y) { p = a.x; break; }
            }
        }
        if (src.s[i] == v) p = v;
        parent[t] = p;
    }
}

template <int K>
cudaError_t parents_k(const uint32_t* in_first, const uint2* in_arc, uint32_t n, const Sources& src,
                      const uint32_t* dist, uint32_t* parent, cudaStream_t st) {
    constexpr uint32_t G = K / RowT<K>::W;
    uint64_t blocks = ((uint64_t)n * G + SWEEP_THREADS - 1) / SWEEP_THREADS;
    blocks = std::min<uint64_t>(blocks, (uint64_t)num_sms() * 8);
    if (blocks == 0) return cudaSuccess;
    parents_kernel<K, false><<<(unsigned)blocks, SWEEP_THREADS, 0, st>>>(in_first, in_arc, nullptr, nullptr, dist, parent,
                                                                      n, src);
    count_launch();
    return cudaGetLastError();
}

// G+ parents (reading R19): one thread per (vertex, tree) item; A-down in-arcs first,
// then A-up in-arcs, the first tight one wins
__global__ void __launch_bounds__(SWEEP_THREADS) parents_ch_kernel(const uint32_t* __restrict__ dn_first,
                                                                   const uint2* __restrict__ dn_arc,
                                                                   const uint32_t* __restrict__ up_first,
                                                                   const uint2* __restrict__ up_arc,
                                                                   const uint32_t* __restrict__ d,
                                                                   uint32_t* __restrict__ parent, uint32_t n,
                                                                   uint32_t k, Sources src) {
    const uint64_t total = (uint64_t)n * k;
    for (uint64_t t = (uint64_t)blockIdx.x * SWEEP_THREADS + threadIdx.x; t < total;
         t += (uint64_t)gridDim.x * SWEEP_THREADS) {
        const uint32_t v = (uint32_t)(t / k), i = (uint32_t)(t % k);
        const uint32_t dv = __ldg(&d[t]);
        uint32_t p = INF;
        if (dv != INF) {
            const uint32_t e1 = __ldg(&dn_first[v + 1]);
            for (uint32_t e = __ldg(&dn_first[v]); e < e1 && p == INF; e++) {
                const uint2 a = __ldg(&dn_arc[e]);
                const uint32_t du = __ldg(&d[(size_t)a.x * k + i]);
                if (du <= dv && dv - du == a.y) p = a.x;
            }
            const uint32_t f1 = __ldg(&up_first[v + 1]);
            for (uint32_t e = __ldg(&up_first[v]); e < f1 && p == INF; e++) {
                const uint2 a = __ldg(&up_arc[e]);
                const uint32_t du = __ldg(&d[(size_t)a.x * k + i]);
                if (du <= dv && dv - du == a.y) p = a.x;
            }
        }
        if (src.s[i] == v) p = v;
        parent[t] = p;
    }
}

}  // namespace

template <int K>
cudaError_t parents_ch_k(const uint32_t* dn_first, const uint2* dn_arc, const uint32_t* upin_first, const uint2* upin_arc,
                         uint32_t n, const Sources& src, const uint32_t* dist, uint32_t* parent, cudaStream_t st) {
    constexpr uint32_t G = K / RowT<K>::W;
    uint64_t blocks = ((uint64_t)n * G + SWEEP_THREADS - 1) / SWEEP_THREADS;
    blocks = std::min<uint64_t>(blocks, (uint64_t)num_sms() * 8);
    if (blocks == 0) return cudaSuccess;
    parents_kernel<K, true><<<(unsigned)blocks, SWEEP_THREADS, 0, st>>>(dn_first, dn_arc, upin_first, upin_arc, dist,
                                                                        parent, n, src);
    count_launch();
    return cudaGetLastError();
}

cudaError_t launch_parents_ch(const uint32_t* dn_first, const uint2* dn_arc, const uint32_t* upin_first,
                              const uint2* upin_arc, uint32_t n, const Sources& src, uint32_t k, const uint32_t* dist,
                              uint32_t* parent, cudaStream_t st) {
    if (k == 1 || k == 2 || k == 4 || k == 8 || k == 16 || k == 32 || k == 64) {
#define CALL_PC(K) parents_ch_k<K>(dn_first, dn_arc, upin_first, upin_arc, n, src, dist, parent, st)
        PHAST_K_SWITCH(k, CALL_PC)
#undef CALL_PC
    }
    uint64_t blocks = ((uint64_t)n * k + SWEEP_THREADS - 1) / SWEEP_THREADS;
    blocks = std::min<uint64_t>(blocks, (uint64_t)num_sms() * 8);
    if (blocks == 0) return cudaSuccess;
    parents_ch_kernel<<<(unsigned)blocks, SWEEP_THREADS, 0, st>>>(dn_first, dn_arc, upin_first, upin_arc, dist, parent,
                                                                  n, k, src);
    count_launch();
    return cudaGetLastError();
}

cudaError_t launch_parents(const uint32_t* in_first, const uint2* in_arc, uint32_t n, const Sources& src,
                           uint32_t k, const uint32_t* dist, uint32_t* parent, cudaStream_t st) {
    if (k == 1 || k == 2 || k == 4 || k == 8 || k == 16 || k == 32 || k == 64) {
#define CALL_PA(K) parents_k<K>(in_first, in_arc, n, src, dist, parent, st)
        PHAST_K_SWITCH(k, CALL_PA)
#undef CALL_PA
    }
    uint64_t blocks = ((uint64_t)n * k + SWEEP_THREADS - 1) / SWEEP_THREADS;
    blocks = std::min<uint64_t>(blocks, (uint64_t)num_sms() * 8);
    if (blocks == 0) return cudaSuccess;
    parents_any_kernel<<<(unsigned)blocks, SWEEP_THREADS, 0, st>>>(in_first, in_arc, dist, parent, n, k, src);
    count_launch();
    return cudaGetLastError();
}

// ------------------------------------------------------------------ NEXT-3 betweenness
// Exact (partial) betweenness on top of k finished trees (§VII-B "c_B(v) =
// sum_{s != v != t} sigma_st(v)/sigma_st").  Rows are [n][k]
// like the labels.  With lengths > 0 the tight arcs d(u) + l = d(w) of a tree form a
// DAG, and sigma (path counts) and delta (Brandes' dependencies) are the unique
// solutions of
//   sigma(v) = [v = s] + sum_{tight (u, v)} sigma(u)
//   delta(v) = sum_{tight (v, w)} sigma(v) / sigma(w) * (1 + delta(w)).
// Every item (v, i) is computed ONCE, in Kahn order of tree i's tight DAG (below), from
// final inputs summed in a fixed arc order, so the result does not depend on the
// schedule.  sigma is an integer held in fp64: exact below 2^53 (the host reports
// ERANGE if any sigma is not finite).  Values written by earlier passes are read with
// plain loads (not __ldg): every pass is a separate launch.
namespace {
__device__ __forceinline__ bool tight(uint32_t du, uint32_t dv, uint32_t l) {
    return du <= dv && dv - du == l;   // du + l == dv without 32-bit overflow
}
// Schedule (not part of the method): Kahn's topological order of each tree's tight DAG.
// Items t = b*nk + v*k + i cover B batches of k trees at once (arrays [B][n][k]): an item
// is computed ONCE, when all its inputs are final: cnt[t] counts the item's unfinished
// inputs (forward: tight in-arcs; backward: tight out-arcs); a pass computes the items
// of its queue and, for each dependent whose count drops to zero, appends it to the
// next queue.  Passes = the largest hop depth of the trees' tight DAGs + 1, so B
// batches share one chain of passes.  Queue sizes rotate over three counters: pass p
// reads qs[p%3], appends with qs[(p+1)%3] and zeroes qs[(p+2)%3].
// warp-aggregated append: the lanes pushing together take consecutive slots with ONE
// atomic (a pass readies up to hundreds of thousands of items: one same-address atomic
// each would serialise the pass)
__device__ __forceinline__ void bc_push(uint32_t t, uint32_t* q, uint32_t* qs, bool& pushed) {
    const unsigned m = __activemask();
    const uint32_t lane = threadIdx.x & 31, leader = __ffs(m) - 1;
    uint32_t base = 0;
    if (lane == leader) base = atomicAdd(qs, (uint32_t)__popc(m));
    base = __shfl_sync(m, base, leader);
    q[base + __popc(m & ((1u << lane) - 1u))] = t;
    pushed = true;
}
// the item of vertex u in item t's tree
__device__ __forceinline__ uint32_t same_tree(uint32_t t, uint32_t v, uint32_t u, uint32_t k) { return t - v * k + u * k; }

// tight-arc masks: bit j of min[t] / mout[t] = the j-th in- / out-arc of item t's vertex
// is tight in t's tree (arcs past the 32nd are re-tested from the labels when used)
__device__ __forceinline__ bool mbit(uint32_t mask, uint32_t j) { return j < 32 ? (mask >> j) & 1u : false; }

// Once per group: the masks of every finite item, then the forward counts (tight in-arcs;
// items with none start queue 0).  The backward counts are popcounts of mout
// (bc_count_back_kernel).
__global__ void __launch_bounds__(256) bc_count_kernel(BcGraph G, const uint32_t* __restrict__ d, uint32_t nk,
                                                       uint32_t k, uint32_t total, uint32_t* cnt, uint32_t* min_,
                                                       uint32_t* mout, uint32_t* q, uint32_t* qs) {
    bool pushed = false;
    for (uint32_t t = blockIdx.x * blockDim.x + threadIdx.x; t < total; t += gridDim.x * blockDim.x) {
        const uint32_t v = (t % nk) / k;
        const uint32_t dv = __ldg(&d[t]);
        if (dv == INF) continue;
        uint32_t c = 0, mi = 0, mo = 0;
        const uint32_t e0 = __ldg(&G.in_first[v]), e1 = __ldg(&G.in_first[v + 1]);
        for (uint32_t e = e0; e < e1; e++) {
            const uint2 a = __ldg(&G.in_arc[e]);
            if (tight(__ldg(&d[same_tree(t, v, a.x, k)]), dv, a.y)) {
                c++;
                if (e - e0 < 32) mi |= 1u << (e - e0);
            }
        }
        const uint32_t f0 = __ldg(&G.out_first[v]), f1 = __ldg(&G.out_first[v + 1]);
        for (uint32_t e = f0; e < f1 && e - f0 < 32; e++) {
            const uint2 a = __ldg(&G.out_arc[e]);
            const uint32_t dw = __ldg(&d[same_tree(t, v, a.x, k)]);
            if (dw != INF && tight(dv, dw, a.y)) mo |= 1u << (e - f0);
        }
        cnt[t] = c;
        min_[t] = mi;
        mout[t] = mo;
        if (c == 0) bc_push(t, q, qs, pushed);
    }
    (void)pushed;
}

// backward counts: tight out-arcs (from mout; past the 32nd from the labels)
__global__ void __launch_bounds__(256) bc_count_back_kernel(BcGraph G, const uint32_t* __restrict__ d, uint32_t nk,
                                                            uint32_t k, uint32_t total, uint32_t* cnt,
                                                            const uint32_t* __restrict__ mout, uint32_t* q,
                                                            uint32_t* qs) {
    bool pushed = false;
    for (uint32_t t = blockIdx.x * blockDim.x + threadIdx.x; t < total; t += gridDim.x * blockDim.x) {
        const uint32_t dv = __ldg(&d[t]);
        if (dv == INF) continue;
        uint32_t c = __popc(__ldg(&mout[t]));
        const uint32_t v = (t % nk) / k;
        const uint32_t f0 = __ldg(&G.out_first[v]), f1 = __ldg(&G.out_first[v + 1]);
        for (uint32_t e = f0 + 32; e < f1; e++) {   // rare: more than 32 out-arcs
            const uint2 a = __ldg(&G.out_arc[e]);
            const uint32_t dw = __ldg(&d[same_tree(t, v, a.x, k)]);
            c += dw != INF && tight(dv, dw, a.y);
        }
        cnt[t] = c;
        if (c == 0) bc_push(t, q, qs, pushed);
    }
    (void)pushed;
}

// Readied dependents: a thread decrements the counts of up to NB dependents of its item
// together (the atomics in flight at once), keeps the ones that reach zero in registers
// and the warp appends all of them with ONE atomic after a warp scan; the loop over the
// queue is warp-uniform so every lane joins the scan.
constexpr uint32_t NB = 8;

struct Ready {
    uint32_t w[NB];
    uint32_t n = 0;
    __device__ __forceinline__ void add(uint32_t x, uint32_t* q, uint32_t* qs, bool& pushed) {
        if (n < NB) {
#pragma unroll
            for (uint32_t j = 0; j < NB; j++)
                if (j == n) w[j] = x;
            n++;
        } else {
            q[atomicAdd(qs, 1u)] = x;   // rare: more than NB readied by one item
            pushed = true;
        }
    }
    // all 32 lanes of the warp call this together
    __device__ __forceinline__ void flush(uint32_t* q, uint32_t* qs, bool& pushed) {
        const uint32_t lane = threadIdx.x & 31;
        uint32_t incl = n;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const uint32_t y = __shfl_up_sync(0xFFFFFFFFu, incl, o);
            if (lane >= (uint32_t)o) incl += y;
        }
        const uint32_t tot = __shfl_sync(0xFFFFFFFFu, incl, 31);
        if (tot == 0) return;
        uint32_t base = 0;
        if (lane == 31) base = atomicAdd(qs, tot);
        base = __shfl_sync(0xFFFFFFFFu, base, 31) + incl - n;
#pragma unroll
        for (uint32_t j = 0; j < NB; j++)
            if (j < n) q[base + j] = w[j];
        pushed = true;
        n = 0;
    }
};

// decrement the counts of the items `dep` of the tight arcs (bits of `mask` over arcs
// [a0, a1) of CSR `arcs`; past the 32nd arc tested from the labels) and collect the
// ones that reach zero
__device__ __forceinline__ void bc_release(const uint2* __restrict__ arcs, uint32_t a0, uint32_t a1, uint32_t mask,
                                           const uint32_t* __restrict__ d, uint32_t t, uint32_t v, uint32_t k,
                                           bool out, uint32_t* cnt, Ready& rd, uint32_t* q, uint32_t* qs,
                                           bool& pushed) {
    for (uint32_t e = a0; e < a1; e += NB) {
        uint32_t w[NB], old[NB];
        bool on[NB];
#pragma unroll
        for (uint32_t j = 0; j < NB; j++) {
            on[j] = false;
            w[j] = 0;
            if (e + j < a1) {
                const uint32_t jj = e + j - a0;
                const uint2 a = __ldg(&arcs[e + j]);
                w[j] = same_tree(t, v, a.x, k);
                if (jj < 32) {
                    on[j] = mbit(mask, jj);
                } else {   // rare: tightness from the labels
                    const uint32_t dt = __ldg(&d[t]), dw = __ldg(&d[w[j]]);
                    on[j] = out ? (dw != INF && tight(dt, dw, a.y)) : tight(dw, dt, a.y);
                }
            }
        }
#pragma unroll
        for (uint32_t j = 0; j < NB; j++) old[j] = on[j] ? atomicSub(&cnt[w[j]], 1u) : 0u;   // in flight together
#pragma unroll
        for (uint32_t j = 0; j < NB; j++)
            if (on[j] && old[j] == 1u) rd.add(w[j], q, qs, pushed);
    }
}

// forward pass: sigma(v) = [v = s] + sum over tight (u, v) of sigma(u).  With lengths > 0
// the source is the only finite item without a tight in-arc, so [v = s] is "no tight
// in-arc" (no source list in the parameters: the passes are graph-captured once per call)
__global__ void __launch_bounds__(256) bc_sigma_kernel(BcGraph G, const uint32_t* __restrict__ d, double* sigma,
                                                       uint32_t nk, uint32_t k, const uint32_t* __restrict__ min_,
                                                       const uint32_t* __restrict__ mout, BcQueue Q,
                                                       uint32_t* changed) {
    const uint32_t size = *Q.qs_in;
    if (blockIdx.x == 0 && threadIdx.x == 0) *Q.qs_clr = 0;
    bool pushed = false;
    Ready rd;
    for (uint32_t x0 = blockIdx.x * blockDim.x; x0 < size; x0 += gridDim.x * blockDim.x) {   // block-uniform
        const uint32_t x = x0 + threadIdx.x;
        if (x < size) {
            const uint32_t t = Q.q_in[x];
            const uint32_t v = (t % nk) / k;
            const uint32_t mi = __ldg(&min_[t]), mo = __ldg(&mout[t]);
            double acc = 0.0;
            bool any = false;
            const uint32_t e0 = __ldg(&G.in_first[v]), e1 = __ldg(&G.in_first[v + 1]);
            for (uint32_t e = e0; e < e1; e++) {
                const bool fast = e - e0 < 32;
                if (fast && !mbit(mi, e - e0)) continue;
                const uint2 a = __ldg(&G.in_arc[e]);
                const uint32_t u = same_tree(t, v, a.x, k);
                if (fast || tight(__ldg(&d[u]), __ldg(&d[t]), a.y)) {
                    acc += sigma[u];
                    any = true;
                }
            }
            if (!(acc <= 9007199254740992.0)) atomicOr(G.err, 1u);   // > 2^53 or not finite: not exact
            sigma[t] = any ? acc : 1.0;
            bc_release(G.out_arc, __ldg(&G.out_first[v]), __ldg(&G.out_first[v + 1]), mo, d, t, v, k, true, Q.cnt, rd,
                       Q.q_out, Q.qs_out, pushed);
        }
        rd.flush(Q.q_out, Q.qs_out, pushed);
    }
    if (__syncthreads_or(pushed) && threadIdx.x == 0) *changed = 1;
}

// backward pass; mode 0: delta(v) = sum over tight (v, w) of sigma(v)/sigma(w) (1 + delta(w));
// mode 1 (reach): height h(v) = max over tight (v, w) of l + h(w), stored as uint32 in
// `val` (l + h(w) <= d(w) + h(w) - d(v) is at most the largest finite label: no wrap)
__global__ void __launch_bounds__(256) bc_back_kernel(BcGraph G, const uint32_t* __restrict__ d,
                                                      const double* __restrict__ sigma, void* val, uint32_t nk,
                                                      uint32_t k, const uint32_t* __restrict__ min_,
                                                      const uint32_t* __restrict__ mout, int mode, BcQueue Q,
                                                      uint32_t* changed) {
    const uint32_t size = *Q.qs_in;
    if (blockIdx.x == 0 && threadIdx.x == 0) *Q.qs_clr = 0;
    bool pushed = false;
    double* delta = static_cast<double*>(val);
    uint32_t* hgt = static_cast<uint32_t*>(val);
    Ready rd;
    for (uint32_t x0 = blockIdx.x * blockDim.x; x0 < size; x0 += gridDim.x * blockDim.x) {   // block-uniform
        const uint32_t x = x0 + threadIdx.x;
        if (x < size) {
            const uint32_t t = Q.q_in[x];
            const uint32_t v = (t % nk) / k;
            const uint32_t mi = __ldg(&min_[t]), mo = __ldg(&mout[t]);
            const uint32_t f0 = __ldg(&G.out_first[v]), f1 = __ldg(&G.out_first[v + 1]);
            double dacc = 0.0;
            uint32_t hacc = 0;
            const double sv = mode == 0 ? __ldg(&sigma[t]) : 0.0;
            for (uint32_t e = f0; e < f1; e++) {
                const bool fast = e - f0 < 32;
                if (fast && !mbit(mo, e - f0)) continue;
                const uint2 a = __ldg(&G.out_arc[e]);
                const uint32_t w = same_tree(t, v, a.x, k);
                if (!fast) {
                    const uint32_t dw = __ldg(&d[w]);
                    if (dw == INF || !tight(__ldg(&d[t]), dw, a.y)) continue;
                }
                if (mode == 0) dacc += sv / __ldg(&sigma[w]) * (1.0 + delta[w]);
                else hacc = max(hacc, a.y + hgt[w]);
            }
            if (mode == 0) delta[t] = dacc; else hgt[t] = hacc;
            bc_release(G.in_arc, __ldg(&G.in_first[v]), __ldg(&G.in_first[v + 1]), mi, d, t, v, k, false, Q.cnt, rd,
                       Q.q_out, Q.qs_out, pushed);
        }
        rd.flush(Q.q_out, Q.qs_out, pushed);
    }
    if (__syncthreads_or(pushed) && threadIdx.x == 0) *changed = 1;
}

// c_B(v) += sum over trees j < valid (j = b*k + i: tree i of batch b) with src[j] != v of
// delta_j(v), in tree order
__global__ void __launch_bounds__(256) bc_accum_kernel(const double* __restrict__ delta, double* __restrict__ cb,
                                                       uint32_t n, uint32_t k, uint32_t valid,
                                                       const uint32_t* __restrict__ src) {
    const uint32_t nk = n * k;
    for (uint32_t v = blockIdx.x * blockDim.x + threadIdx.x; v < n; v += gridDim.x * blockDim.x) {
        double s = 0.0;
        for (uint32_t j = 0; j < valid; j++)
            if (__ldg(&src[j]) != v) s += __ldg(&delta[(size_t)(j / k) * nk + (size_t)v * k + j % k]);
        cb[v] += s;
    }
}

// r(v) = max(r(v), max over trees j < valid of min(d_j(v), h_j(v)))
__global__ void __launch_bounds__(256) reach_accum_kernel(const uint32_t* __restrict__ d,
                                                          const uint32_t* __restrict__ hgt, uint32_t* __restrict__ r,
                                                          uint32_t n, uint32_t k, uint32_t valid) {
    const uint32_t nk = n * k;
    for (uint32_t v = blockIdx.x * blockDim.x + threadIdx.x; v < n; v += gridDim.x * blockDim.x) {
        uint32_t m = r[v];
        for (uint32_t j = 0; j < valid; j++) {
            const size_t t = (size_t)(j / k) * nk + (size_t)v * k + j % k;
            const uint32_t dv = __ldg(&d[t]);
            if (dv != INF) m = max(m, min(dv, __ldg(&hgt[t])));
        }
        r[v] = m;
    }
}

unsigned bc_blocks(uint64_t items) {
    uint64_t b = (items + 255) / 256;
    return (unsigned)std::max<uint64_t>(1, std::min<uint64_t>(b, (uint64_t)num_sms() * 8));
}

// the passes touch only their queue (its size is read on the device): a full wave
unsigned bc_pass_blocks(uint64_t items) { return bc_blocks(items); }

}  // namespace

cudaError_t launch_bc_count(const BcGraph& G, const uint32_t* d, uint32_t nk, uint32_t k, uint32_t total, int backward,
                            uint32_t* cnt, uint32_t* min_, uint32_t* mout, uint32_t* q, uint32_t* qs, cudaStream_t st) {
    if (backward)
        bc_count_back_kernel<<<bc_blocks(total), 256, 0, st>>>(G, d, nk, k, total, cnt, mout, q, qs);
    else
        bc_count_kernel<<<bc_blocks(total), 256, 0, st>>>(G, d, nk, k, total, cnt, min_, mout, q, qs);
    count_launch();
    return cudaGetLastError();
}

cudaError_t launch_bc_sigma(const BcGraph& G, const uint32_t* d, double* sigma, uint32_t nk, uint32_t k,
                            uint32_t total, const uint32_t* min_, const uint32_t* mout, const BcQueue& Q,
                            uint32_t* changed, cudaStream_t st) {
    bc_sigma_kernel<<<bc_pass_blocks(total), 256, 0, st>>>(G, d, sigma, nk, k, min_, mout, Q, changed);
    count_launch();
    return cudaGetLastError();
}

cudaError_t launch_bc_back(const BcGraph& G, const uint32_t* d, const double* sigma, void* val, uint32_t nk,
                           uint32_t k, uint32_t total, const uint32_t* min_, const uint32_t* mout, int mode,
                           const BcQueue& Q, uint32_t* changed, cudaStream_t st) {
    bc_back_kernel<<<bc_pass_blocks(total), 256, 0, st>>>(G, d, sigma, val, nk, k, min_, mout, mode, Q, changed);
    count_launch();
    return cudaGetLastError();
}

cudaError_t launch_reach_accum(const uint32_t* d, const uint32_t* hgt, uint32_t* r, uint32_t n, uint32_t k,
                               uint32_t valid, cudaStream_t st) {
    reach_accum_kernel<<<bc_blocks(n), 256, 0, st>>>(d, hgt, r, n, k, valid);
    count_launch();
    return cudaGetLastError();
}

cudaError_t launch_bc_accum(const double* delta, double* cb, uint32_t n, uint32_t k, uint32_t valid,
                            const uint32_t* src, cudaStream_t st) {
    bc_accum_kernel<<<bc_blocks(n), 256, 0, st>>>(delta, cb, n, k, valid, src);
    count_launch();
    return cudaGetLastError();
}

}  // namespace phast
