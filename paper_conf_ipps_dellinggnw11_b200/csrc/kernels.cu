// kernels.cu -- PHAST's hot path on sm_100a.
//
// a1 upward CH search  : one CTA per source, exact labels in G-up by label-correcting
//                        relaxation over a shared-memory hash table (global fallback).
//                        PAPER.md:14 §III "it runs Dijkstra's algorithm from s in G-up,
//                        stopping when the priority queue becomes empty"; any method
//                        giving exact G-up distances is valid (reading R9).
// a2 seed + implicit init: visited bits (§IV-C "we mark vertices visited
//                        during the CH search with a single bit"), rows of the search
//                        space reset to INF, then labels scattered (two launches so
//                        every reset precedes every scatter).
// a3 downward sweep    : per level, d(v) = min(flag(v) ? d(v) : INF,
//                        min_{(u,v) in A-down} sat(d(u) + l(u,v))) for k trees at once
//                        (§III, §IV-B).  k/4 lanes per vertex,
//                        16-byte label loads per lane (the B200 analogue of "four trees
//                        per SSE register", §IV-B).
// a5 diameter          : max over finite labels fused into the sweep (PAPER.md:20
//                        §VII-B "making each core keep track of the maximum label it
//                        encounters").
// No tensor cores: the loop is an integer (min,+) gather with no reuse.
#include <algorithm>
#include <atomic>
#include <cstdio>
#include <vector>
#include <cstdlib>

#include <cooperative_groups.h>
#include "kernels.h"

namespace phast {

static std::atomic<uint64_t> g_launches{0};
// L2 persistence window over the first rows of the label array (the top levels, which
// a level-by-level sweep re-reads once per lower level holding one of their heads):
// bytes, 0 = off (set_l2_persist)
static size_t g_persist_bytes = 0;
uint64_t launches() { return g_launches.load(); }
void add_launches(int64_t d) { g_launches += (uint64_t)d; }

int set_l2_persist(size_t bytes) {
    if (bytes) {
        int dev = 0, maxw = 0, maxp = 0;
        if (cudaGetDevice(&dev) != cudaSuccess ||
            cudaDeviceGetAttribute(&maxw, cudaDevAttrMaxAccessPolicyWindowSize, dev) != cudaSuccess ||
            cudaDeviceGetAttribute(&maxp, cudaDevAttrMaxPersistingL2CacheSize, dev) != cudaSuccess) {
            cudaGetLastError();
            return -1;
        }
        bytes = std::min<size_t>(bytes, std::min<size_t>((size_t)maxw, (size_t)maxp));
        if (cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, bytes) != cudaSuccess) {
            cudaGetLastError();
            return -1;
        }
    }
    g_persist_bytes = bytes;
    return 0;
}

int num_sms() {
    static int sms = 0;
    if (!sms) {
        int dev = 0;
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
        if (sms <= 0) sms = 148;
    }
    return sms;
}

namespace {

constexpr uint32_t EMPTY = 0xFFFFFFFFu;
constexpr int UP_THREADS = 512;
constexpr uint32_t UP_SMEM_CAP = 4096;   // shared-memory table entries per source

__device__ __forceinline__ uint32_t sat_add(uint32_t a, uint32_t l) {
    // min(a + l, INF) without wrap: min(a, INF - l) + l   (reading R1)
    return min(a, INF - l) + l;
}
__device__ __forceinline__ uint32_t hash32(uint32_t x) {
    x ^= x >> 16; x *= 0x7feb352dU; x ^= x >> 15; x *= 0x846ca68bU; x ^= x >> 16;
    return x;
}

// ------------------------------------------------------------------ a1 upward
struct UpTable {
    uint32_t* keys;
    uint32_t* vals;
    uint32_t* inq;
    uint32_t* qa;
    uint32_t* qb;
    uint32_t cap;  // power of two
};

struct UpShared {
    uint32_t qn, nn, used, over, cnt;
};

// Returns the slot of w (inserting it), or EMPTY when the table is 3/4 full.
__device__ __forceinline__ uint32_t up_insert(const UpTable& t, uint32_t w, UpShared& c) {
    uint32_t mask = t.cap - 1;
    uint32_t h = hash32(w) & mask;
    for (uint32_t probe = 0; probe < t.cap; probe++) {
        uint32_t k = *((volatile uint32_t*)&t.keys[h]);
        if (k == w) return h;
        if (k == EMPTY) {
            if (atomicAdd(&c.used, 0u) * 4 >= t.cap * 3) return EMPTY;
            uint32_t old = atomicCAS(&t.keys[h], EMPTY, w);
            if (old == EMPTY) { atomicAdd(&c.used, 1u); return h; }
            if (old == w) return h;
        }
        h = (h + 1) & mask;
    }
    return EMPTY;
}

// Label-correcting relaxation of G-up from s, wave-synchronous; on return the
// table holds exact G-up distances of every vertex reachable from s (Bellman-Ford
// fixed point with saturating sums).  Returns false on table overflow.
// vtop > 0: vertices < vtop (the top levels, swept by sweep_top_kernel's G-up pull
// pass) get their labels from the arcs entering them but are not expanded.
__device__ bool up_search(const uint32_t* __restrict__ up_first, const uint2* __restrict__ up_arc,
                          uint32_t s, UpTable t, UpShared& c, uint32_t vtop) {
    const uint32_t tid = threadIdx.x;
    for (uint32_t i = tid; i < t.cap; i += blockDim.x) { t.keys[i] = EMPTY; t.vals[i] = INF; t.inq[i] = 0; }
    __syncthreads();
    if (tid == 0) {
        uint32_t h = hash32(s) & (t.cap - 1);
        t.keys[h] = s; t.vals[h] = 0; t.inq[h] = 1; t.qa[0] = h;
        c.qn = s >= vtop ? 1u : 0u; c.nn = 0; c.used = 1; c.over = 0; c.cnt = 0;
    }
    __syncthreads();
    uint32_t* qa = t.qa;
    uint32_t* qb = t.qb;
    for (;;) {
        uint32_t qn = c.qn;
        if (qn == 0 || c.over) break;
        for (uint32_t idx = tid; idx < qn; idx += blockDim.x) {
            uint32_t slot = qa[idx];
            atomicExch(&t.inq[slot], 0u);
            __threadfence_block();
            uint32_t v = t.keys[slot];
            uint32_t dv = *((volatile uint32_t*)&t.vals[slot]);
            uint32_t e1 = __ldg(&up_first[v + 1]);
            for (uint32_t e = __ldg(&up_first[v]); e < e1; e++) {
                uint2 a = __ldg(&up_arc[e]);
                uint32_t nd = sat_add(dv, a.y);
                if (nd == INF) continue;
                uint32_t ws = up_insert(t, a.x, c);
                if (ws == EMPTY) { c.over = 1; break; }
                uint32_t old = atomicMin(&t.vals[ws], nd);
                if (nd < old && a.x >= vtop) {
                    __threadfence_block();
                    if (atomicExch(&t.inq[ws], 1u) == 0u) qb[atomicAdd(&c.nn, 1u)] = ws;
                }
            }
        }
        __syncthreads();
        if (tid == 0) { c.qn = c.nn; c.nn = 0; }
        uint32_t* tmp = qa; qa = qb; qb = tmp;
        __syncthreads();
    }
    bool ok = !c.over;
    __syncthreads();
    return ok;
}

// a1: search only; the search space goes to seed slot `slot` (the sweep of the
// previous batch may still be running on the main stream: nothing here touches the
// visited bits or the label rows).
__global__ void __launch_bounds__(UP_THREADS) upward_kernel(DevImage g, Sources src, uint32_t slot, uint32_t vtop) {
    extern __shared__ uint32_t smem[];
    __shared__ UpShared c;
    const uint32_t i = blockIdx.x;
    const uint32_t s = src.s[i];
    const uint32_t sc = g.smem_cap;
    const size_t so = ((size_t)slot * KMAX + i) * g.seed_cap;
    UpTable t{smem, smem + sc, smem + 2 * sc, smem + 3 * sc, smem + 4 * sc, sc};
    bool ok = up_search(g.up_first, g.up_arc, s, t, c, vtop);
    if (!ok) {   // global-memory fallback with the per-source capacity
        uint32_t* base = g.gscratch + (size_t)i * g.seed_cap * 5;
        UpTable gt{base, base + g.seed_cap, base + 2 * (size_t)g.seed_cap, base + 3 * (size_t)g.seed_cap,
                   base + 4 * (size_t)g.seed_cap, g.seed_cap};
        t = gt;
        ok = up_search(g.up_first, g.up_arc, s, t, c, vtop);
        if (!ok) {
            if (threadIdx.x == 0) { atomicOr(g.err, 1u); g.seed_cnt[slot * KMAX + i] = 0; }
            return;
        }
    }
    uint32_t* sv = g.seed_v + so;
    uint32_t* sd = g.seed_d + so;
    for (uint32_t e = threadIdx.x; e < t.cap; e += blockDim.x) {
        uint32_t v = t.keys[e];
        if (v == EMPTY) continue;
        uint32_t pos = atomicAdd(&c.cnt, 1u);
        sv[pos] = v;
        sd[pos] = t.vals[e];
    }
    __syncthreads();
    if (threadIdx.x == 0) g.seed_cnt[slot * KMAX + i] = c.cnt;
}

// a2 phase 1: visited bits of the search space, and its rows reset to INF
template <int K>
__global__ void seed_rows_kernel(DevImage g, uint32_t slot, uint32_t* __restrict__ dist) {
    const uint32_t i = blockIdx.x;
    const uint32_t cnt = g.seed_cnt[slot * KMAX + i];
    const uint32_t* sv = g.seed_v + ((size_t)slot * KMAX + i) * g.seed_cap;
    for (uint32_t j = threadIdx.x; j < cnt; j += blockDim.x) {
        const uint32_t v = sv[j];
        atomicOr(&g.flags[v >> 5], 1u << (v & 31));
    }
    if constexpr (K % 4 == 0) {
        constexpr uint32_t W = K / 4;
        const uint4 inf4 = make_uint4(INF, INF, INF, INF);
        for (uint32_t j = threadIdx.x; j < cnt * W; j += blockDim.x)
            reinterpret_cast<uint4*>(dist + (size_t)sv[j / W] * K)[j % W] = inf4;
    } else {
        for (uint32_t j = threadIdx.x; j < cnt * K; j += blockDim.x) dist[(size_t)sv[j / K] * K + j % K] = INF;
    }
}

// a2 phase 2 (after every reset of phase 1): the labels
__global__ void scatter_kernel(DevImage g, uint32_t slot, uint32_t k, uint32_t* __restrict__ dist) {
    const uint32_t i = blockIdx.x;
    const uint32_t cnt = g.seed_cnt[slot * KMAX + i];
    const uint32_t* sv = g.seed_v + ((size_t)slot * KMAX + i) * g.seed_cap;
    const uint32_t* sd = g.seed_d + ((size_t)slot * KMAX + i) * g.seed_cap;
    for (uint32_t j = threadIdx.x; j < cnt; j += blockDim.x) dist[(size_t)sv[j] * k + i] = sd[j];
}

__global__ void clear_flags_kernel(DevImage g, uint32_t slot) {
    const uint32_t i = blockIdx.x;
    const uint32_t cnt = g.seed_cnt[slot * KMAX + i];
    const uint32_t* sv = g.seed_v + ((size_t)slot * KMAX + i) * g.seed_cap;
    for (uint32_t j = threadIdx.x; j < cnt; j += blockDim.x) g.flags[sv[j] >> 5] = 0u;
}

// ------------------------------------------------------------------ a3 sweep
template <int K> struct RowT;
template <> struct RowT<1> { using T = uint32_t; static constexpr int W = 1; };
template <> struct RowT<2> { using T = uint2; static constexpr int W = 2; };
template <int K> struct RowT { using T = uint4; static constexpr int W = 4; };

__device__ __forceinline__ uint32_t vinf(uint32_t) { return INF; }
__device__ __forceinline__ uint32_t relax(uint32_t acc, uint32_t x, uint32_t l) { return min(acc, sat_add(x, l)); }
__device__ __forceinline__ uint2 relax(uint2 acc, uint2 x, uint32_t l) {
    uint32_t c = INF - l;
    return make_uint2(min(acc.x, min(x.x, c) + l), min(acc.y, min(x.y, c) + l));
}
__device__ __forceinline__ uint4 relax(uint4 acc, uint4 x, uint32_t l) {
    uint32_t c = INF - l;
    return make_uint4(min(acc.x, min(x.x, c) + l), min(acc.y, min(x.y, c) + l),
                      min(acc.z, min(x.z, c) + l), min(acc.w, min(x.w, c) + l));
}
__device__ __forceinline__ uint32_t fmax_of(uint32_t a) { return a == INF ? 0u : a; }
__device__ __forceinline__ uint32_t fmax_of(uint2 a) { return max(fmax_of(a.x), fmax_of(a.y)); }
__device__ __forceinline__ uint32_t fmax_of(uint4 a) {
    return max(max(fmax_of(a.x), fmax_of(a.y)), max(fmax_of(a.z), fmax_of(a.w)));
}
template <class T> __device__ __forceinline__ T inf_row();
template <> __device__ __forceinline__ uint32_t inf_row<uint32_t>() { return INF; }
template <> __device__ __forceinline__ uint2 inf_row<uint2>() { return make_uint2(INF, INF); }
template <> __device__ __forceinline__ uint4 inf_row<uint4>() { return make_uint4(INF, INF, INF, INF); }

template <class T> __device__ __forceinline__ void st_stream(T* p, T v) { __stcs(p, v); }

constexpr int SWEEP_THREADS = 256;
constexpr int ELL = 16;   // sweep_kernel AB value: ELL-2 records (DevImage::dn_rec) instead of the CSR
constexpr int ELLP = 17;  // ELL-2 records, the next item's record loaded one item ahead

// One level [vbeg, vend) (§VI "The CPU starts, for each level i, a kernel on
// the GPU").  One (vertex, 16-byte lane) item per thread per grid-stride step; the
// grid fills every SM (8 CTAs of 256 threads), which keeps the most gathers in flight
// (measured: a two-items-per-thread variant with fewer resident CTAs was 30 % slower
// on level 0, profiles/r1_launches_*).  Launched with programmatic dependent launch:
// the next level's grid is launched while this one drains and blocks in
// griddepcontrol.wait until this grid's rows are visible.
// TB (segments that mix levels): per vertex, tails are stored normally (re-read soon,
// from L2) and the other rows with evict-first stores (diameter: not stored at all).
// AB > 1: up to AB arcs of the item (then their AB tail rows) are loaded together,
// so an item costs two dependent round trips after its offsets, not 2 * degree.
template <int K, bool DIAM, bool STORE, bool STREAM, bool TB, int AB>
__global__ void __launch_bounds__(SWEEP_THREADS, AB >= 3 && AB < 8 ? 6 : 8) sweep_kernel(const uint32_t* __restrict__ first,
                                                               const uint2* __restrict__ arcs,
                                                               const uint4* __restrict__ rec,
                                                               const uint2* __restrict__ ovf,
                                                               uint32_t* __restrict__ d,
                                                               const uint32_t* __restrict__ flags,
                                                               const uint32_t* __restrict__ tail_bits,
                                                               uint32_t vbeg, uint32_t vend,
                                                               uint32_t* __restrict__ diam) {
    using T = typename RowT<K>::T;
    constexpr uint32_t W = RowT<K>::W;
    constexpr uint32_t G = K / W;   // lanes per vertex
    asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
    const uint32_t total = (vend - vbeg) * G;   // host: < 2^31 (sweep_launch splits longer segments)
    // The graph (offsets, arcs) is static: the first item's offsets are loaded and its
    // first arcs prefetched into L2 BEFORE griddepcontrol.wait, overlapping the previous
    // level's drain; only label rows (flags, tail rows) must wait.  The loop itself
    // re-reads them (L1 / L2 hits) so that it keeps its register budget.
    uint32_t t = blockIdx.x * SWEEP_THREADS + threadIdx.x;
    uint4 rn = make_uint4(INF, INF, INF, INF);   // ELLP: the next item's record, loaded one item ahead
    if (t < total) {
        if constexpr (AB == ELLP) {
            rn = __ldg(&rec[vbeg + t / G]);
        } else if constexpr (AB == ELL) {
            asm volatile("prefetch.global.L2 [%0];" ::"l"(rec + vbeg + t / G));
        } else {
            const uint32_t e0 = __ldg(&first[vbeg + t / G]);
            asm volatile("prefetch.global.L2 [%0];" ::"l"(arcs + e0));
        }
    }
    asm volatile("griddepcontrol.wait;" ::: "memory");          // previous level complete and visible
    uint32_t mx = 0;
    for (; t < total; t += gridDim.x * SWEEP_THREADS) {
        const uint32_t v = vbeg + t / G;
        const uint32_t lane = t % G;
        T acc = inf_row<T>();
        if ((__ldg(&flags[v >> 5]) >> (v & 31)) & 1u)   // visited by an upward search
            acc = __ldg(reinterpret_cast<const T*>(d + (size_t)v * K) + lane);
        if constexpr (AB == ELL || AB == ELLP) {
            // one 16-byte record: the vertex's first two in-arcs (97 % of level-0 and
            // 92 % of level-1 vertices have at most two), so the gather depends on ONE
            // load instead of offsets -> arcs
            // (a missing arc has len INF: relaxing an INF row by it changes nothing)
            uint4 r;
            if constexpr (AB == ELLP) {   // record loaded one item ahead: the gathers wait on nothing
                r = rn;
                const uint32_t tn = t + gridDim.x * SWEEP_THREADS;
                if (tn < total) rn = __ldg(&rec[vbeg + tn / G]);
            } else {
                r = __ldg(&rec[v]);
            }
            T x0 = inf_row<T>(), x1 = inf_row<T>();
            if (r.y != INF) x0 = __ldg(reinterpret_cast<const T*>(d + (size_t)r.x * K) + lane);
            if (r.w != INF) x1 = __ldg(reinterpret_cast<const T*>(d + (size_t)r.z * K) + lane);
            acc = relax(relax(acc, x0, r.y), x1, r.w);
            if (r.w == INF && r.z != INF) {   // more than two in-arcs: the rest in the overflow list
                const uint2* o = ovf + r.z;
                const uint32_t cnt = __ldg(&o->x);
                for (uint32_t j = 1; j <= cnt; j++) {
                    const uint2 a = __ldg(&o[j]);
                    acc = relax(acc, __ldg(reinterpret_cast<const T*>(d + (size_t)a.x * K) + lane), a.y);
                }
            }
        } else {
        const uint32_t e0 = __ldg(&first[v]), e1 = __ldg(&first[v + 1]);
        if constexpr (AB == 1) {
#pragma unroll 4
            for (uint32_t e = e0; e < e1; e++) {
                const uint2 a = __ldg(&arcs[e]);
                const T x = __ldg(reinterpret_cast<const T*>(d + (size_t)a.x * K) + lane);
                acc = relax(acc, x, a.y);
            }
        } else if constexpr (AB >= 8 && RowT<K>::W == 4) {
            // AB = 8: four arcs per batch, their tail rows copied into shared memory by
            // cp.async (no registers held by loads in flight), then reduced from there
            __shared__ __align__(16) uint4 srow[4][SWEEP_THREADS];
            for (uint32_t e = e0; e < e1; e += 4) {
                uint2 a[4];
#pragma unroll
                for (int r = 0; r < 4; r++)
                    if (e + r < e1) a[r] = __ldg(&arcs[e + r]);
#pragma unroll
                for (int r = 0; r < 4; r++)
                    if (e + r < e1)
                        asm volatile("cp.async.ca.shared.global [%0], [%1], 16;" ::"r"(
                                         static_cast<uint32_t>(__cvta_generic_to_shared(&srow[r][threadIdx.x]))),
                                     "l"(reinterpret_cast<const uint4*>(d + (size_t)a[r].x * K) + lane)
                                     : "memory");
                asm volatile("cp.async.commit_group;\ncp.async.wait_group 0;" ::: "memory");
#pragma unroll
                for (int r = 0; r < 4; r++)
                    if (e + r < e1) acc = relax(acc, srow[r][threadIdx.x], a[r].y);
            }
        } else {
            for (uint32_t e = e0; e < e1; e += (AB >= 8 ? 4 : AB)) {
                constexpr int B = AB >= 8 ? 4 : AB;
                uint2 a[B];
                T x[B];
#pragma unroll
                for (int r = 0; r < B; r++)
                    if (e + r < e1) a[r] = __ldg(&arcs[e + r]);
#pragma unroll
                for (int r = 0; r < B; r++)
                    if (e + r < e1) x[r] = __ldg(reinterpret_cast<const T*>(d + (size_t)a[r].x * K) + lane);
#pragma unroll
                for (int r = 0; r < B; r++)
                    if (e + r < e1) acc = relax(acc, x[r], a[r].y);
            }
        }
        }   // CSR path
        if constexpr (TB) {
            T* p = reinterpret_cast<T*>(d + (size_t)v * K) + lane;
            if ((__ldg(&tail_bits[v >> 5]) >> (v & 31)) & 1u) *p = acc;
            else if constexpr (!DIAM) st_stream(p, acc);
        } else if constexpr (STORE) {
            T* p = reinterpret_cast<T*>(d + (size_t)v * K) + lane;
            if constexpr (STREAM) st_stream(p, acc); else *p = acc;
        }
        if constexpr (DIAM) mx = max(mx, fmax_of(acc));
    }
    if constexpr (DIAM) {
        __shared__ uint32_t wmax[SWEEP_THREADS / 32];
        mx = __reduce_max_sync(0xFFFFFFFFu, mx);
        if ((threadIdx.x & 31) == 0) wmax[threadIdx.x >> 5] = mx;
        __syncthreads();
        if (threadIdx.x < 32) {
            uint32_t w = threadIdx.x < SWEEP_THREADS / 32 ? wmax[threadIdx.x] : 0u;
            w = __reduce_max_sync(0xFFFFFFFFu, w);
            if (threadIdx.x == 0 && w) atomicMax(diam, w);
        }
    }
}

int arc_batch() {   // PHAST_ARC_BATCH: 1, 2, 3, 4, 8 (staged) or 16 (ELL-2 records, default); read per launch
    const char* e = std::getenv("PHAST_ARC_BATCH");
    int b = e ? std::atoi(e) : ELL;
    if (b != 8 && b != ELL && b != ELLP && (b < 1 || b > 4)) b = ELL;
    return b;
}

template <int K, bool DIAM, bool STORE, bool STREAM, bool TB>
cudaError_t sweep_launch(const DevImage& g, uint32_t vbeg, uint32_t vend, uint32_t* dist, uint32_t* diam,
                         cudaStream_t st) {
    constexpr uint32_t G = K / RowT<K>::W;
    constexpr uint32_t VMAX = (1u << 31) / G;   // 32-bit item indices in the kernel
    if (vend - vbeg > VMAX) {                    // a level has no internal arcs: split it freely
        cudaError_t e = sweep_launch<K, DIAM, STORE, STREAM, TB>(g, vbeg, vbeg + VMAX, dist, diam, st);
        return e != cudaSuccess ? e : sweep_launch<K, DIAM, STORE, STREAM, TB>(g, vbeg + VMAX, vend, dist, diam, st);
    }
    uint64_t total = (uint64_t)(vend - vbeg) * G;
    uint64_t blocks = (total + SWEEP_THREADS - 1) / SWEEP_THREADS;
    int ab = arc_batch();
    if ((ab == ELL || ab == ELLP) && !g.dn_rec) ab = 2;
    // one full wave of resident CTAs (the kernels' launch bounds: 8, 6 for AB 3-4)
    const uint64_t cap = (uint64_t)num_sms() * ((ab == 3 || ab == 4) ? 6 : 8);
    if (blocks > cap) blocks = cap;
    if (blocks == 0) return cudaSuccess;
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3((unsigned)blocks);
    cfg.blockDim = dim3(SWEEP_THREADS);
    cfg.dynamicSmemBytes = 0;
    cfg.stream = st;
    cudaLaunchAttribute attr[2];
    attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    if (g_persist_bytes) {   // the top levels' rows (ids [0, ...): re-read by many lower levels) persist in L2
        attr[1].id = cudaLaunchAttributeAccessPolicyWindow;
        attr[1].val.accessPolicyWindow.base_ptr = dist;
        attr[1].val.accessPolicyWindow.num_bytes = std::min<size_t>(g_persist_bytes, (size_t)vend * K * 4);
        attr[1].val.accessPolicyWindow.hitRatio = 1.0f;
        attr[1].val.accessPolicyWindow.hitProp = cudaAccessPropertyPersisting;
        attr[1].val.accessPolicyWindow.missProp = cudaAccessPropertyStreaming;
        cfg.numAttrs = 2;
    }
    cudaError_t e = cudaLaunchKernelEx(&cfg, ab == ELLP ? sweep_kernel<K, DIAM, STORE, STREAM, TB, ELLP>
                                             : ab == ELL ? sweep_kernel<K, DIAM, STORE, STREAM, TB, ELL>
                                             : ab == 8 ? sweep_kernel<K, DIAM, STORE, STREAM, TB, 8>
                                             : ab == 4 ? sweep_kernel<K, DIAM, STORE, STREAM, TB, 4>
                                             : ab == 3 ? sweep_kernel<K, DIAM, STORE, STREAM, TB, 3>
                                             : ab == 2 ? sweep_kernel<K, DIAM, STORE, STREAM, TB, 2>
                                                       : sweep_kernel<K, DIAM, STORE, STREAM, TB, 1>,
                                       g.dn_first, g.dn_arc, g.dn_rec, g.dn_ovf, dist, (const uint32_t*)g.flags,
                                       g.tail_bits, vbeg, vend, diam);
    g_launches++;
    return e;
}

template <int K>
cudaError_t sweep_k(const DevImage& g, uint32_t vbeg, uint32_t vend, uint32_t* dist, uint32_t* diam, bool store,
                    bool last, bool by_tail, cudaStream_t st) {
    if (by_tail)
        return diam ? sweep_launch<K, true, true, false, true>(g, vbeg, vend, dist, diam, st)
                    : sweep_launch<K, false, true, false, true>(g, vbeg, vend, dist, diam, st);
    if (diam) {
        if (!store) return sweep_launch<K, true, false, false, false>(g, vbeg, vend, dist, diam, st);
        return last ? sweep_launch<K, true, true, true, false>(g, vbeg, vend, dist, diam, st)
                    : sweep_launch<K, true, true, false, false>(g, vbeg, vend, dist, diam, st);
    }
    return last ? sweep_launch<K, false, true, true, false>(g, vbeg, vend, dist, diam, st)
                : sweep_launch<K, false, true, false, false>(g, vbeg, vend, dist, diam, st);
}

// ------------------------------------------------------------------ NEXT-1 parent pointers
// After a sweep every label is final, so the parent pass has no dependencies: one
// grid-stride pass over (vertex, 16-byte lane) items.  Each lane owns W trees of the
// row; it scans v's original in-arcs in input order and keeps, per tree, the tail of
// the first tight arc (§VII-A).  The identity is tested as d(u) <= d(v)
// and d(v) - d(u) = l, which equals d(u) + l = d(v) exactly (no 32-bit overflow).
// The scan stops once every finite tree of the lane has its parent.
template <int K>
__global__ void __launch_bounds__(SWEEP_THREADS) parents_kernel(const uint32_t* __restrict__ in_first,
                                                                const uint2* __restrict__ in_arc,
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
        const uint32_t e1 = __ldg(&in_first[v + 1]);
        for (uint32_t e = __ldg(&in_first[v]); need && e < e1; e++) {
            const uint2 a = __ldg(&in_arc[e]);
            const T ru = __ldg(reinterpret_cast<const T*>(d + (size_t)a.x * K) + lane);
            const uint32_t* du = reinterpret_cast<const uint32_t*>(&ru);
#pragma unroll
            for (uint32_t q = 0; q < W; q++)
                if (((need >> q) & 1u) && du[q] <= dv[q] && dv[q] - du[q] == a.y) {
                    p[q] = a.x;
                    need &= ~(1u << q);
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

template <int K>
cudaError_t parents_k(const uint32_t* in_first, const uint2* in_arc, uint32_t n, const Sources& src,
                      const uint32_t* dist, uint32_t* parent, cudaStream_t st) {
    constexpr uint32_t G = K / RowT<K>::W;
    uint64_t blocks = ((uint64_t)n * G + SWEEP_THREADS - 1) / SWEEP_THREADS;
    blocks = std::min<uint64_t>(blocks, (uint64_t)num_sms() * 8);
    if (blocks == 0) return cudaSuccess;
    parents_kernel<K><<<(unsigned)blocks, SWEEP_THREADS, 0, st>>>(in_first, in_arc, dist, parent, n, src);
    g_launches++;
    return cudaGetLastError();
}

// ------------------------------------------------------------------ a3+a4 persistent sweep
// ONE launch for the whole sweep.  The internal order is topological (layout.cpp),
// so the sweep is "a simple linear sweep in increasing order of IDs" (PAPER.md:16
// §IV-A), cut into chunks of consecutive ids.  CTA b takes chunks b, b+grid, ...; a
// chunk waits until every CTA has finished the iteration that produced its latest
// tail (per-iteration completion counters, release/acquire at gpu scope), replacing
// the paper's kernel launch per level (§VI).  STAGE: each chunk's
// offsets first[vbeg..vend] and its contiguous G-down arc block are moved into shared
// memory by the bulk-copy engine (cp.async.bulk + mbarrier), double-buffered: the
// copy for the CTA's next chunk is in flight while the current chunk gathers, so a
// gather waits on one HBM/L2 round trip (the tail row), not two.
constexpr uint32_t CHUNK_PASSES = 4;     // passes of the CTA over G-lane vertex groups per chunk
constexpr uint32_t STAGE_ARCS = 1024;    // arcs per shared-memory buffer (8 KB)

__device__ __forceinline__ uint32_t ld_acquire_gpu(const uint32_t* p) {
    uint32_t v;
    asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
// Completion-flag read for the kernels whose label reads all bypass L1 (ld.global.cg /
// cp.async.cg, served by L2, the GPU's point of coherence): a relaxed read suffices
// in practice -- the producer's rows reach L2 before its release-store of the flag,
// and every row load is issued only after the flag value has been observed (control
// dependency).  An acquire load would also invalidate the SM's whole L1 (CCTL.IVALL)
// on every check, which ncu showed costing ~13 % of the warp-pipelined sweep's stalls.
__device__ __forceinline__ uint32_t ld_flag(const uint32_t* p) {
    uint32_t v;
    asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_release_gpu(uint32_t* p, uint32_t v) {
    asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ uint64_t globaltimer_ns() {
    uint64_t t;
    asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
    return t;
}
__device__ __forceinline__ uint32_t smem_u32(const void* p) {
    return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}
__device__ __forceinline__ void cp_async16(void* smem, const void* gmem) {
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(smem_u32(smem)), "l"(gmem) : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
__device__ __forceinline__ void cp_async_wait_all() { asm volatile("cp.async.wait_group 0;" ::: "memory"); }
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_arrive_tx(uint64_t* bar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t phase) {
    asm volatile(
        "{\n"
        ".reg .pred P1;\n"
        "WAIT_%=:\n"
        "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n"
        "@!P1 bra WAIT_%=;\n"
        "}\n" ::"r"(smem_u32(bar)),
        "r"(phase)
        : "memory");
}
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                     smem_u32(dst)),
                 "l"(src), "r"(bytes), "r"(smem_u32(bar))
                 : "memory");
}

struct StageInfo {
    uint32_t vbeg, vend, dep;   // chunk [vbeg, vend); dep = 1 + iteration to wait for (0 = none)
    uint32_t f0;                // vertex id of sfirst[0] (multiple of 4)
    uint32_t a0;                // arc index of sarc[0] (even)
    uint32_t staged;            // 1 if first/arcs are in shared memory
};

template <int K, bool DIAM, bool STAGE>
__global__ void __launch_bounds__(SWEEP_THREADS, 4) sweep_persistent_kernel(const uint32_t* __restrict__ first,
                                                                            const uint2* __restrict__ arcs,
                                                                            uint32_t* __restrict__ d,
                                                                            const uint32_t* __restrict__ flags,
                                                                            const uint32_t* __restrict__ tail_bits,
                                                                            SweepPlan p, uint32_t epoch,
                                                                            uint32_t* __restrict__ diam) {
    using T = typename RowT<K>::T;
    constexpr uint32_t W = RowT<K>::W;
    constexpr uint32_t G = K / W;                               // lanes per vertex
    constexpr uint32_t VPP = SWEEP_THREADS / G;                 // vertices per pass
    constexpr uint32_t STAGE_FIRST = VPP * CHUNK_PASSES + 8;    // first[vbeg..vend], 16-byte aligned
    __shared__ __align__(16) uint2 sarc[STAGE ? 2 : 1][STAGE ? STAGE_ARCS : 2];
    __shared__ __align__(16) uint32_t sfirst[STAGE ? 2 : 1][STAGE ? STAGE_FIRST : 4];
    __shared__ __align__(8) uint64_t bar[2];
    __shared__ StageInfo info[2];
    __shared__ uint32_t s_known;                                // leading iterations known complete
    const uint32_t grid = gridDim.x;
    const uint32_t lane = threadIdx.x % G;
    if (threadIdx.x == 0) {
        s_known = 0;
        if constexpr (STAGE) {
            mbar_init(&bar[0], 1);
            mbar_init(&bar[1], 1);
            asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
        }
    }
    __syncthreads();

    // thread 0: describe chunk c in info[b] and start its bulk copies
    auto stage = [&](uint32_t b, uint32_t c) {
        StageInfo in;
        in.vbeg = __ldg(&p.chunk_v[c]);
        in.vend = __ldg(&p.chunk_v[c + 1]);
        in.dep = __ldg(&p.chunk_dep[c]);
        in.f0 = in.vbeg & ~3u;
        in.a0 = 0;
        in.staged = 0;
        if constexpr (STAGE) {
            const uint32_t f1 = (in.vend + 1 + 3) & ~3u;      // [f0, f1) covers first[vbeg..vend]
            const uint32_t e0 = __ldg(&first[in.vbeg]), e1 = __ldg(&first[in.vend]);
            in.a0 = e0 & ~1u;
            const uint32_t a1 = (e1 + 1) & ~1u;
            if (f1 - in.f0 <= STAGE_FIRST && a1 - in.a0 <= STAGE_ARCS) {
                in.staged = 1;
                asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
                const uint32_t fb = (f1 - in.f0) * 4, ab = (a1 - in.a0) * 8;
                mbar_arrive_tx(&bar[b], fb + ab);
                bulk_g2s(&sfirst[b][0], first + in.f0, fb, &bar[b]);
                if (ab) bulk_g2s(&sarc[b][0], arcs + in.a0, ab, &bar[b]);
            }
        }
        info[b] = in;
    };

    uint32_t phase = 0;   // bit b = parity of the next completion of bar[b]
    uint32_t mx = 0;
    if (threadIdx.x == 0 && blockIdx.x < p.nchunks) stage(0, blockIdx.x);
    uint32_t it = 0;
    for (uint32_t c = blockIdx.x; c < p.nchunks; c += grid, it++) {
        const uint32_t b = it & 1u;
        if (threadIdx.x == 0) {
            const uint32_t dep = info[b].dep;
            if (dep > s_known) {                               // wait for iteration dep-1 everywhere
                const uint32_t w = dep - 1;
                const uint32_t need = epoch * min(grid, p.nchunks - w * grid);
                uint32_t ns = 32;
                const uint64_t t0 = globaltimer_ns();
                while (ld_acquire_gpu(&p.wave_done[w]) < need) {
                    __nanosleep(ns);
                    ns = min(ns * 2, 256u);
                    if ((*(volatile uint32_t*)p.err & 2u) || globaltimer_ns() - t0 > 4000000000ull) {
                        atomicOr(p.err, 2u);                        // watchdog: never hang the GPU;
                        break;                                      // phast_sync reports ECUDA
                    }
                }
                s_known = dep;                                 // counters are monotone in w
                __threadfence();                               // drop older L1 lines of this SM
            }
        }
        __syncthreads();
        const StageInfo in = info[b];
        if (threadIdx.x == 0 && c + grid < p.nchunks) stage(b ^ 1u, c + grid);   // prefetch the next chunk
        if (STAGE && in.staged) {
            mbar_wait(&bar[b], (phase >> b) & 1u);
            phase ^= 1u << b;
        }
        for (uint32_t base = in.vbeg; base < in.vend; base += VPP) {
            const uint32_t v = base + threadIdx.x / G;
            if (v >= in.vend) break;
            T acc = inf_row<T>();
            if ((__ldg(&flags[v >> 5]) >> (v & 31)) & 1u)   // visited by an upward search (§IV-C)
                acc = reinterpret_cast<const T*>(d + (size_t)v * K)[lane];
            uint32_t e, e1;
            if (STAGE && in.staged) {
                e = sfirst[b][v - in.f0];
                e1 = sfirst[b][v + 1 - in.f0];
            } else {
                e = __ldg(&first[v]);
                e1 = __ldg(&first[v + 1]);
            }
            while (e < e1) {                                   // up to 4 gathers in flight per lane
                const uint32_t cnt = min(e1 - e, 4u);
                uint2 a[4];
                T x[4];
#pragma unroll
                for (uint32_t j = 0; j < 4; j++)
                    if (j < cnt) a[j] = (STAGE && in.staged) ? sarc[b][e + j - in.a0] : __ldg(&arcs[e + j]);
#pragma unroll
                for (uint32_t j = 0; j < 4; j++)
                    if (j < cnt) x[j] = reinterpret_cast<const T*>(d + (size_t)a[j].x * K)[lane];
#pragma unroll
                for (uint32_t j = 0; j < 4; j++)
                    if (j < cnt) acc = relax(acc, x[j], a[j].y);
                e += cnt;
            }
            const bool is_tail = (__ldg(&tail_bits[v >> 5]) >> (v & 31)) & 1u;
            if (!DIAM || is_tail) {                            // diameter: rows nobody reads are not stored
                T* q = reinterpret_cast<T*>(d + (size_t)v * K) + lane;
                if (is_tail) *q = acc;                         // re-read soon from L2
                else st_stream(q, acc);                        // never re-read: evict first
            }
            if constexpr (DIAM) mx = max(mx, fmax_of(acc));
        }
        __syncthreads();                                       // every row of this chunk is written
        if (threadIdx.x == 0) {
            __threadfence();                                   // release: rows before the counter
            atomicAdd(&p.wave_done[it], 1u);
        }
    }
    if constexpr (DIAM) {
        __shared__ uint32_t wmax[SWEEP_THREADS / 32];
        mx = __reduce_max_sync(0xFFFFFFFFu, mx);
        if ((threadIdx.x & 31) == 0) wmax[threadIdx.x >> 5] = mx;
        __syncthreads();
        if (threadIdx.x < 32) {
            uint32_t w = threadIdx.x < SWEEP_THREADS / 32 ? wmax[threadIdx.x] : 0u;
            w = __reduce_max_sync(0xFFFFFFFFu, w);
            if (threadIdx.x == 0 && w) atomicMax(diam, w);
        }
    }
}

// ------------------------------------------------------------------ a3+a4 warp dataflow (variant 2)
// ONE launch; the unit of work is a chunk of consecutive ids handled by ONE warp.
// Chunk c runs on warp c % workers; before gathering, the warp's lanes acquire the
// completion flags of the chunks holding its tails (precomputed list, only chunks of
// other warps).  No CTA barriers, no level or wave coupling: a chunk starts as soon
// as its own tails are final.  Label rows are read with ld.global.cg (L2), never
// from a possibly stale L1 line.
constexpr uint32_t WARP_PASSES = 4;
constexpr uint32_t WARP_STAGE_ARCS = 64;
constexpr uint32_t WARPS_PER_CTA = SWEEP_THREADS / 32;

template <int K, bool DIAM>
__global__ void __launch_bounds__(SWEEP_THREADS, 5) sweep_warp_kernel(const uint32_t* __restrict__ first,
                                                                      const uint2* __restrict__ arcs,
                                                                      uint32_t* __restrict__ d,
                                                                      const uint32_t* __restrict__ flags,
                                                                      const uint32_t* __restrict__ tail_bits,
                                                                      SweepPlan p, uint32_t epoch,
                                                                      uint32_t* __restrict__ diam) {
    using T = typename RowT<K>::T;
    constexpr uint32_t W = RowT<K>::W;
    constexpr uint32_t G = K / W;              // lanes per vertex
    constexpr uint32_t VPW = 32 / G;           // vertices per warp pass
    constexpr uint32_t CAP = VPW * WARP_PASSES;
    __shared__ uint2 sarc[WARPS_PER_CTA][WARP_STAGE_ARCS];
    __shared__ uint32_t sfirst[WARPS_PER_CTA][CAP + 1];
    const uint32_t wid = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const uint32_t gl = lane % G, grp = lane / G;
    uint32_t mx = 0;
    for (uint32_t c = blockIdx.x * WARPS_PER_CTA + wid; c < p.nchunks; c += p.workers) {
        uint4 m = __ldg(&p.wmeta[c]);          // {vbeg, vend, dbeg, dend | bit 31}
        m.w &= 0x7FFFFFFFu;
        for (uint32_t i = m.z + lane; i < m.w; i += 32) {
            const uint32_t x = __ldg(&p.wdeps[i]);
            if (ld_acquire_gpu(&p.done[x]) < epoch) {
                uint32_t ns = 32;
                const uint64_t t0 = globaltimer_ns();
                while (ld_acquire_gpu(&p.done[x]) < epoch) {
                    __nanosleep(ns);
                    ns = min(ns * 2, 512u);
                    if ((*(volatile uint32_t*)p.err & 2u) || globaltimer_ns() - t0 > 4000000000ull) {
                        atomicOr(p.err, 2u);                       // watchdog: never hang the GPU
                        break;
                    }
                }
            }
        }
        __syncwarp();
        const uint32_t nv = m.y - m.x;
        for (uint32_t i = lane; i <= nv; i += 32) sfirst[wid][i] = __ldg(&first[m.x + i]);
        __syncwarp();
        const uint32_t e0 = sfirst[wid][0];
        const uint32_t na = sfirst[wid][nv] - e0;
        const bool staged = na <= WARP_STAGE_ARCS;
        if (staged)
            for (uint32_t i = lane; i < na; i += 32) sarc[wid][i] = __ldg(&arcs[e0 + i]);
        __syncwarp();
        for (uint32_t base = 0; base < nv; base += VPW) {
            const uint32_t li = base + grp;
            if (li >= nv) break;
            const uint32_t v = m.x + li;
            T acc = inf_row<T>();
            if ((__ldg(&flags[v >> 5]) >> (v & 31)) & 1u)   // visited by an upward search (§IV-C)
                acc = __ldcg(reinterpret_cast<const T*>(d + (size_t)v * K) + gl);
            uint32_t e = sfirst[wid][li];
            const uint32_t e1 = sfirst[wid][li + 1];
            while (e < e1) {                                   // up to 4 gathers in flight per lane
                const uint32_t cnt = min(e1 - e, 4u);
                uint2 a[4];
                T x[4];
#pragma unroll
                for (uint32_t j = 0; j < 4; j++)
                    if (j < cnt) a[j] = staged ? sarc[wid][e + j - e0] : __ldg(&arcs[e + j]);
#pragma unroll
                for (uint32_t j = 0; j < 4; j++)
                    if (j < cnt) x[j] = __ldcg(reinterpret_cast<const T*>(d + (size_t)a[j].x * K) + gl);
#pragma unroll
                for (uint32_t j = 0; j < 4; j++)
                    if (j < cnt) acc = relax(acc, x[j], a[j].y);
                e += cnt;
            }
            const bool is_tail = (__ldg(&tail_bits[v >> 5]) >> (v & 31)) & 1u;
            if (!DIAM || is_tail) {                            // diameter: rows nobody reads are not stored
                T* q = reinterpret_cast<T*>(d + (size_t)v * K) + gl;
                if (is_tail) *q = acc;                         // re-read soon, from L2
                else st_stream(q, acc);                        // never re-read: evict first
            }
            if constexpr (DIAM) mx = max(mx, fmax_of(acc));
        }
        __syncwarp();                                          // all rows of the chunk are issued
        if (lane == 0) st_release_gpu(&p.done[c], epoch);     // release: cumulative over the warp
    }
    if constexpr (DIAM) {
        mx = __reduce_max_sync(0xFFFFFFFFu, mx);
        if (lane == 0 && mx) atomicMax(diam, mx);
    }
}

// ------------------------------------------------------------------ a3+a4 warp pipeline (variant 4)
// Warp dataflow (as variant 2) with a software pipeline inside each warp: the chunk
// descriptors and dependency ids are loaded two chunks ahead, the chunk's offsets
// and arc block are copied into shared memory by cp.async one chunk ahead (three
// rotating buffers), so the per-chunk critical path is one acquire of the producers'
// completion flags (usually already set) plus one round trip of tail-row gathers.
constexpr uint32_t WP_ARCS = 128;

template <int K>
struct WpGeom {
    static constexpr uint32_t W = RowT<K>::W;
    static constexpr uint32_t G = K / W;
    static constexpr uint32_t VPW = 32 / G;
    static constexpr uint32_t CAP = VPW * 4 < 32 ? VPW * 4 : 32;
    static constexpr uint32_t FCAP = CAP + 8;
};

template <int K, bool DIAM>
__global__ void __launch_bounds__(SWEEP_THREADS, 4) sweep_wpipe_kernel(const uint32_t* __restrict__ first,
                                                                       const uint2* __restrict__ arcs,
                                                                       uint32_t* __restrict__ d,
                                                                       const uint32_t* __restrict__ flags,
                                                                       const uint32_t* __restrict__ tail_bits,
                                                                       SweepPlan p, uint32_t epoch,
                                                                       uint32_t* __restrict__ diam) {
    using T = typename RowT<K>::T;
    using Geo = WpGeom<K>;
    constexpr uint32_t G = Geo::G, VPW = Geo::VPW, FCAP = Geo::FCAP;
    __shared__ __align__(16) uint2 sarc[WARPS_PER_CTA][3][WP_ARCS];
    __shared__ __align__(16) uint32_t sfirst[WARPS_PER_CTA][3][FCAP];
    const uint32_t wid = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const uint32_t gl = lane % G, grp = lane / G;
    const uint32_t NW = p.workers;
    uint32_t mx = 0;

    auto stage = [&](uint32_t buf, const uint4& in) {   // cp.async offsets + arc block of a chunk
        const uint32_t f0 = in.x & ~3u, f1 = (in.y + 1 + 3) & ~3u;
        for (uint32_t i = lane; i < (f1 - f0) / 4; i += 32) cp_async16(&sfirst[wid][buf][i * 4], first + f0 + i * 4);
        const uint32_t a0 = in.z & ~1u, a1 = (in.w + 1) & ~1u;
        if (a1 - a0 <= WP_ARCS)
            for (uint32_t i = lane; i < (a1 - a0) / 2; i += 32) cp_async16(&sarc[wid][buf][i * 2], arcs + a0 + i * 2);
        cp_async_commit();
    };
    auto load_dep = [&](uint32_t c) -> uint2 {          // {dbeg, dend & flag}
        return __ldg(reinterpret_cast<const uint2*>(&p.wmeta[c]) + 1);
    };

    uint32_t c = blockIdx.x * WARPS_PER_CTA + wid;
    uint4 in_c = make_uint4(0, 0, 0, 0), in_n = in_c, in_nn = in_c;
    uint2 dr_c = make_uint2(0, 0), dr_n = dr_c, dr_nn = dr_c;
    uint32_t did_c = 0, did_n = 0;                       // this lane's first dependency id
    if (c < p.nchunks) {
        in_c = __ldg(&p.pinfo[c]);
        dr_c = load_dep(c);
        if (dr_c.x + lane < (dr_c.y & 0x7FFFFFFFu)) did_c = __ldg(&p.wdeps[dr_c.x + lane]);
        stage(0, in_c);
        if (c + NW < p.nchunks) {
            in_n = __ldg(&p.pinfo[c + NW]);
            dr_n = load_dep(c + NW);
            if (dr_n.x + lane < (dr_n.y & 0x7FFFFFFFu)) did_n = __ldg(&p.wdeps[dr_n.x + lane]);
            stage(1, in_n);
        } else {
            cp_async_commit();
        }
    }
    uint32_t bc = 0;
    for (; c < p.nchunks; c += NW) {
        const uint32_t cn = c + NW, cnn = cn + NW;
        if (cnn < p.nchunks) { in_nn = __ldg(&p.pinfo[cnn]); dr_nn = load_dep(cnn); }
        // 1. producers of c: acquire their completion flags
        {
            const uint32_t dend = dr_c.y & 0x7FFFFFFFu;
            for (uint32_t i = dr_c.x + lane; i < dend; i += 32) {
                const uint32_t x = (i == dr_c.x + lane) ? did_c : __ldg(&p.wdeps[i]);
                if (ld_flag(&p.done[x]) < epoch) {
                    uint32_t ns = 32;
                    const uint64_t t0 = globaltimer_ns();
                    while (ld_flag(&p.done[x]) < epoch) {
                        __nanosleep(ns);
                        ns = min(ns * 2, 256u);
                        if ((*(volatile uint32_t*)p.err & 2u) || globaltimer_ns() - t0 > 4000000000ull) {
                            atomicOr(p.err, 2u);   // watchdog: report, never hang
                            break;
                        }
                    }
                }
            }
        }
        // 2. offsets and arcs of c are in shared memory (stage of cn may still fly)
        asm volatile("cp.async.wait_group 1;" ::: "memory");
        __syncwarp();
        const uint32_t* sf = sfirst[wid][bc];
        const uint2* sa = sarc[wid][bc];
        const uint32_t f0 = in_c.x & ~3u, a0 = in_c.z & ~1u;
        const bool staged = ((in_c.w + 1) & ~1u) - a0 <= WP_ARCS;
        const uint32_t nv = in_c.y - in_c.x;
        for (uint32_t base = 0; base < nv; base += VPW) {
            const uint32_t li = base + grp;
            if (li >= nv) break;
            const uint32_t v = in_c.x + li;
            T acc = inf_row<T>();
            if ((__ldg(&flags[v >> 5]) >> (v & 31)) & 1u)   // visited by an upward search (§IV-C)
                acc = __ldcg(reinterpret_cast<const T*>(d + (size_t)v * K) + gl);
            uint32_t e = sf[v - f0];
            const uint32_t e1 = sf[v + 1 - f0];
            while (e < e1) {                                   // up to 4 gathers in flight per lane
                const uint32_t cnt = min(e1 - e, 4u);
                uint2 a[4];
                T x[4];
#pragma unroll
                for (uint32_t j = 0; j < 4; j++)
                    if (j < cnt) a[j] = staged ? sa[e + j - a0] : __ldg(&arcs[e + j]);
#pragma unroll
                for (uint32_t j = 0; j < 4; j++)
                    if (j < cnt) x[j] = __ldcg(reinterpret_cast<const T*>(d + (size_t)a[j].x * K) + gl);
#pragma unroll
                for (uint32_t j = 0; j < 4; j++)
                    if (j < cnt) acc = relax(acc, x[j], a[j].y);
                e += cnt;
            }
            const bool is_tail = (__ldg(&tail_bits[v >> 5]) >> (v & 31)) & 1u;
            if (!DIAM || is_tail) {
                T* q = reinterpret_cast<T*>(d + (size_t)v * K) + gl;
                if (is_tail) *q = acc; else st_stream(q, acc);
            }
            if constexpr (DIAM) mx = max(mx, fmax_of(acc));
        }
        __syncwarp();
        if (lane == 0) st_release_gpu(&p.done[c], epoch);     // release: cumulative over the warp
        // 3. lookahead: dependency ids of cn's successor, staging of cnn
        uint32_t did_nn = 0;
        if (cnn < p.nchunks) {
            if (dr_nn.x + lane < (dr_nn.y & 0x7FFFFFFFu)) did_nn = __ldg(&p.wdeps[dr_nn.x + lane]);
            stage((bc + 2) % 3, in_nn);
        } else {
            cp_async_commit();
        }
        in_c = in_n; dr_c = dr_n; did_c = did_n;
        in_n = in_nn; dr_n = dr_nn; did_n = did_nn;
        bc = (bc + 1) % 3;
    }
    asm volatile("cp.async.wait_group 0;" ::: "memory");
    if constexpr (DIAM) {
        mx = __reduce_max_sync(0xFFFFFFFFu, mx);
        if (lane == 0 && mx) atomicMax(diam, mx);
    }
}

template <int K, bool DIAM>
int wpipe_occupancy() {
    int b = 0;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, sweep_wpipe_kernel<K, DIAM>, SWEEP_THREADS, 0) !=
        cudaSuccess) {
        cudaGetLastError();
        return 1;
    }
    return b > 0 ? b : 1;
}

template <int K, bool DIAM>
int warp_occupancy() {
    int b = 0;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, sweep_warp_kernel<K, DIAM>, SWEEP_THREADS, 0) !=
        cudaSuccess) {
        cudaGetLastError();
        return 1;
    }
    return b > 0 ? b : 1;
}

// ------------------------------------------------------------------ a3+a4 warp waves (variant 5)
// ONE launch; T = gridDim.x * 8 warps, every one resident.  Warp w runs slots w, w+T,
// w+2T, ... of the wave plan (layout.cpp: plan_waves), so slot j*T + w is its j-th
// chunk and "wave j" is the j-th chunk of every warp.  A warp finishes its chunks in
// order, hence "wave j complete" (all T warps signalled j) implies every wave < j is
// complete: a chunk waits on ONE condition, the wave of its latest tail chunk, which
// the plan puts strictly before the chunk's own wave (§III "(For
// correctness, any reverse topological order will do.)").  A warp caches how many
// leading waves it knows to be complete, so in the bulk of the wavefront (tails about
// delta ids, i.e. several waves, back) a check costs nothing.
// Completion: 8 sub-counters per wave (warp w adds to w % 8), monotone over launches
// (each reaches T/8 * epoch), spread over separate 256-byte lines.
// Per warp, the chunk's offsets and arc block are staged into shared memory by
// cp.async one chunk ahead, the descriptors two ahead; inside a chunk every lane owns
// STEPS (vertex, 16-byte lane) items and issues the first WAVE_R gathers of all of
// them before reducing any (up to STEPS*WAVE_R 16-byte loads in flight per lane).
constexpr uint32_t WAVE_STEPS = 4;
constexpr uint32_t WAVE_R = 2;          // gathers per item issued together
constexpr uint32_t WAVE_ACAP = 64;      // staged arcs per chunk
constexpr uint32_t WAVE_SUB = 8;        // sub-counters per wave

template <int K>
struct WaveGeom {
    static constexpr uint32_t G = K / RowT<K>::W;        // lanes per row
    static constexpr uint32_t VPS = 32 / G;              // vertices per warp step
    static constexpr uint32_t U = VPS * WAVE_STEPS;      // vertices per chunk (<= 128)
    static constexpr uint32_t FCAP = U + 8;              // staged offsets (16-byte aligned window)
};

template <int K, bool DIAM>
__global__ void __launch_bounds__(SWEEP_THREADS, 2) sweep_wave_kernel(const uint32_t* __restrict__ first,
                                                                      const uint2* __restrict__ arcs,
                                                                      uint32_t* __restrict__ d,
                                                                      const uint32_t* __restrict__ flags,
                                                                      const uint32_t* __restrict__ tail_bits,
                                                                      SweepPlan p, uint32_t epoch,
                                                                      uint32_t* __restrict__ diam) {
    using T = typename RowT<K>::T;
    using Geo = WaveGeom<K>;
    constexpr uint32_t G = Geo::G, VPS = Geo::VPS, FCAP = Geo::FCAP;
    __shared__ __align__(16) uint2 sarc[WARPS_PER_CTA][2][WAVE_ACAP];
    __shared__ __align__(16) uint32_t sfirst[WARPS_PER_CTA][2][FCAP];
    const uint32_t wid = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const uint32_t gl = lane % G, grp = lane / G;
    const uint32_t NT = p.workers;                       // T
    const uint32_t w = blockIdx.x * WARPS_PER_CTA + wid;
    const uint32_t nw = p.iters;                         // waves
    const uint32_t stride = p.chunk_cap;                 // sub-counter stride (words)
    const uint32_t target = (NT / WAVE_SUB) * epoch;
    const uint4* __restrict__ desc = p.wdesc;
    uint32_t* cnt = p.wave_done;
    uint32_t mx = 0;

    auto stage = [&](uint32_t buf, const uint4& in) {   // cp.async offsets + arc block of a chunk
        const uint32_t vn = in.y & 0xFFu;
        if (vn) {
            const uint32_t f0 = in.x & ~3u, f1 = (in.x + vn + 1 + 3) & ~3u;
            for (uint32_t i = lane; i < (f1 - f0) / 4; i += 32) cp_async16(&sfirst[wid][buf][i * 4], first + f0 + i * 4);
            const uint32_t a0 = in.z & ~1u, a1 = (in.w + 1) & ~1u;
            if (a1 - a0 <= WAVE_ACAP)
                for (uint32_t i = lane; i < (a1 - a0) / 2; i += 32) cp_async16(&sarc[wid][buf][i * 2], arcs + a0 + i * 2);
        }
        cp_async_commit();
    };

    const uint4 zero = make_uint4(0, 0, 0, 0);
    uint4 in_c = nw > 0 ? __ldg(&desc[w]) : zero;
    uint4 in_n = nw > 1 ? __ldg(&desc[(size_t)NT + w]) : zero;
    stage(0, in_c);
    uint32_t known = 0;                                  // waves [0, known) are complete
    for (uint32_t j = 0; j < nw; j++) {
        const uint4 in_nn = j + 2 < nw ? __ldg(&desc[(size_t)(j + 2) * NT + w]) : zero;
        stage((j + 1) & 1, in_n);
        // 1. the wave holding this chunk's latest tail must be complete
        const uint32_t dep1 = in_c.y >> 8;
        if (dep1 > known) {
            const uint32_t x = dep1 - 1;
            bool ok = lane >= WAVE_SUB || ld_flag(&cnt[(size_t)lane * stride + x]) >= target;
            if (!__all_sync(0xFFFFFFFFu, ok)) {
                uint32_t ns = 32;
                const uint64_t t0 = globaltimer_ns();
                for (;;) {
                    __nanosleep(ns);
                    ns = min(ns * 2, 256u);
                    ok = lane >= WAVE_SUB || ld_flag(&cnt[(size_t)lane * stride + x]) >= target;
                    if (__all_sync(0xFFFFFFFFu, ok)) break;
                    bool dead = lane == 0 && ((*(volatile uint32_t*)p.err & 2u) ||
                                              globaltimer_ns() - t0 > 4000000000ull);
                    if (__any_sync(0xFFFFFFFFu, dead)) {
                        if (lane == 0) atomicOr(p.err, 2u);   // watchdog: report, never hang
                        break;
                    }
                }
            }
            known = dep1;
        }
        // 2. this chunk's offsets and arcs are in shared memory (the next chunk's may fly)
        asm volatile("cp.async.wait_group 1;" ::: "memory");
        __syncwarp();
        const uint32_t vn = in_c.y & 0xFFu;
        if (vn) {
            const uint32_t* sf = sfirst[wid][j & 1];
            const uint2* sa = sarc[wid][j & 1];
            const uint32_t f0 = in_c.x & ~3u, a0 = in_c.z & ~1u;
            const bool staged = ((in_c.w + 1) & ~1u) - a0 <= WAVE_ACAP;
            uint32_t v[WAVE_STEPS], e[WAVE_STEPS], e1[WAVE_STEPS];
            T acc[WAVE_STEPS];
#pragma unroll
            for (uint32_t s = 0; s < WAVE_STEPS; s++) {
                const uint32_t li = s * VPS + grp;
                v[s] = in_c.x + li;
                acc[s] = inf_row<T>();
                e[s] = e1[s] = 0;
                if (li < vn) {
                    if ((__ldg(&flags[v[s] >> 5]) >> (v[s] & 31)) & 1u)   // visited (§IV-C)
                        acc[s] = __ldcg(reinterpret_cast<const T*>(d + (size_t)v[s] * K) + gl);
                    e[s] = sf[v[s] - f0];
                    e1[s] = sf[v[s] + 1 - f0];
                }
            }
            {   // first round: WAVE_R gathers of every item in flight together
                uint2 a[WAVE_STEPS][WAVE_R];
                T x[WAVE_STEPS][WAVE_R];
#pragma unroll
                for (uint32_t s = 0; s < WAVE_STEPS; s++)
#pragma unroll
                    for (uint32_t r = 0; r < WAVE_R; r++)
                        if (e[s] + r < e1[s]) a[s][r] = staged ? sa[e[s] + r - a0] : __ldg(&arcs[e[s] + r]);
#pragma unroll
                for (uint32_t s = 0; s < WAVE_STEPS; s++)
#pragma unroll
                    for (uint32_t r = 0; r < WAVE_R; r++)
                        if (e[s] + r < e1[s]) x[s][r] = __ldcg(reinterpret_cast<const T*>(d + (size_t)a[s][r].x * K) + gl);
#pragma unroll
                for (uint32_t s = 0; s < WAVE_STEPS; s++)
#pragma unroll
                    for (uint32_t r = 0; r < WAVE_R; r++)
                        if (e[s] + r < e1[s]) acc[s] = relax(acc[s], x[s][r], a[s][r].y);
            }
#pragma unroll
            for (uint32_t s = 0; s < WAVE_STEPS; s++) {   // the rest (high in-degree vertices)
                for (uint32_t q = e[s] + WAVE_R; q < e1[s]; q += 4) {
                    const uint32_t c = min(e1[s] - q, 4u);
                    uint2 a[4];
                    T x[4];
#pragma unroll
                    for (uint32_t r = 0; r < 4; r++)
                        if (r < c) a[r] = staged ? sa[q + r - a0] : __ldg(&arcs[q + r]);
#pragma unroll
                    for (uint32_t r = 0; r < 4; r++)
                        if (r < c) x[r] = __ldcg(reinterpret_cast<const T*>(d + (size_t)a[r].x * K) + gl);
#pragma unroll
                    for (uint32_t r = 0; r < 4; r++)
                        if (r < c) acc[s] = relax(acc[s], x[r], a[r].y);
                }
            }
#pragma unroll
            for (uint32_t s = 0; s < WAVE_STEPS; s++) {
                if (s * VPS + grp >= vn) continue;
                const bool is_tail = (__ldg(&tail_bits[v[s] >> 5]) >> (v[s] & 31)) & 1u;
                if (!DIAM || is_tail) {                          // diameter: rows nobody reads are not stored
                    T* q = reinterpret_cast<T*>(d + (size_t)v[s] * K) + gl;
                    if (is_tail) *q = acc[s];                    // re-read soon, from L2
                    else st_stream(q, acc[s]);                   // never re-read: evict first
                }
                if constexpr (DIAM) mx = max(mx, fmax_of(acc[s]));
            }
        }
        // 3. signal wave j: every lane's rows are performed at gpu scope, then one add
        __threadfence();
        __syncwarp();
        if (lane == 0)
            asm volatile("red.relaxed.gpu.global.add.u32 [%0], 1;" ::"l"(&cnt[(size_t)(w % WAVE_SUB) * stride + j])
                         : "memory");
        in_c = in_n;
        in_n = in_nn;
    }
    asm volatile("cp.async.wait_group 0;" ::: "memory");
    if constexpr (DIAM) {
        mx = __reduce_max_sync(0xFFFFFFFFu, mx);
        if (lane == 0 && mx) atomicMax(diam, mx);
    }
}

template <int K, bool DIAM>
int wave_occupancy() {
    int b = 0;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, sweep_wave_kernel<K, DIAM>, SWEEP_THREADS, 0) !=
        cudaSuccess) {
        cudaGetLastError();
        return 1;
    }
    return b > 0 ? b : 1;
}

// ------------------------------------------------------------------ a3+a4 segment barriers (variant 6)
// ONE launch for a segmented layout (levels, or the diagonal layout's levels +
// diagonals; layout.h: lvl_off): the grid walks the segments in order, each one
// exactly like one per-level launch (grid-stride (vertex, 16-byte lane) items,
// PAPER.md:18 §VI), and meets at a grid-wide barrier between segments -- the
// paper's kernel boundary between levels (§VI "The CPU starts, for each
// level i, a kernel on the GPU") without its launch and drain cost.  The barrier is
// one arrival per CTA on a per-segment counter (monotone over launches: it reaches
// grid * epoch) and an acquire spin by thread 0, which also drops the SM's L1 lines
// (tail rows are read with plain L1-cached loads; the lines of rows finalised in
// the segment just completed may be stale there).  All CTAs are resident (grid
// sized by the occupancy calculator); a 4 s watchdog turns a stuck barrier into
// PHAST_ECUDA instead of a hang.
// BATCH: the next item's offsets are prefetched while the current one gathers, and
// up to 4 arcs (then their 4 tail rows) are loaded together: two dependent round
// trips per item instead of 1 + 2 * degree.
template <int K, bool DIAM, bool BATCH>
__global__ void __launch_bounds__(SWEEP_THREADS, BATCH ? 6 : 8) sweep_seg_kernel(const uint32_t* __restrict__ first,
                                                                  const uint2* __restrict__ arcs,
                                                                  uint32_t* __restrict__ d,
                                                                  const uint32_t* __restrict__ flags,
                                                                  const uint32_t* __restrict__ tail_bits,
                                                                  SweepPlan p, uint32_t epoch,
                                                                  uint32_t* __restrict__ diam) {
    using T = typename RowT<K>::T;
    constexpr uint32_t G = K / RowT<K>::W;   // lanes per vertex
    const uint32_t nseg = p.nchunks, tb_from = p.chunk_cap;
    const uint32_t target = gridDim.x * epoch;
    const uint32_t stride = gridDim.x * SWEEP_THREADS;   // host: n * G < 2^31
    uint32_t mx = 0;
    uint32_t vb = __ldg(&p.chunk_v[0]);
    for (uint32_t j = 0; j < nseg; j++) {
        const uint32_t ve = __ldg(&p.chunk_v[j + 1]);
        const bool tb = j >= tb_from, last = p.stream_last && j + 1 == nseg;
        const uint32_t total = (ve - vb) * G;
        uint32_t t = blockIdx.x * SWEEP_THREADS + threadIdx.x;
        uint32_t nf0 = 0, nf1 = 0;
        if (BATCH && t < total) {
            const uint32_t v = vb + (t / G);
            nf0 = __ldg(&first[v]);
            nf1 = __ldg(&first[v + 1]);
        }
        for (; t < total; t += stride) {
            const uint32_t v = vb + (t / G);
            const uint32_t lane = (t % G);
            T acc = inf_row<T>();
            if ((__ldg(&flags[v >> 5]) >> (v & 31)) & 1u)   // visited by an upward search (§IV-C)
                acc = __ldcg(reinterpret_cast<const T*>(d + (size_t)v * K) + lane);
            if constexpr (BATCH) {
                const uint32_t e0 = nf0, e1 = nf1;
                if (t + stride < total) {                    // prefetch the next item's offsets
                    const uint32_t vn = vb + ((t + stride) / G);
                    nf0 = __ldg(&first[vn]);
                    nf1 = __ldg(&first[vn + 1]);
                }
                for (uint32_t e = e0; e < e1; e += 4) {
                    uint2 a[4];
                    T x[4];
#pragma unroll
                    for (uint32_t r = 0; r < 4; r++)
                        if (e + r < e1) a[r] = __ldg(&arcs[e + r]);
#pragma unroll
                    for (uint32_t r = 0; r < 4; r++)
                        if (e + r < e1) x[r] = __ldca(reinterpret_cast<const T*>(d + (size_t)a[r].x * K) + lane);
#pragma unroll
                    for (uint32_t r = 0; r < 4; r++)
                        if (e + r < e1) acc = relax(acc, x[r], a[r].y);
                }
            } else {
                const uint32_t e0 = __ldg(&first[v]), e1 = __ldg(&first[v + 1]);
#pragma unroll 4
                for (uint32_t e = e0; e < e1; e++) {
                    const uint2 a = __ldg(&arcs[e]);
                    const T x = __ldca(reinterpret_cast<const T*>(d + (size_t)a.x * K) + lane);
                    acc = relax(acc, x, a.y);
                }
            }
            T* q = reinterpret_cast<T*>(d + (size_t)v * K) + lane;
            if (tb) {
                if ((__ldg(&tail_bits[v >> 5]) >> (v & 31)) & 1u) *q = acc;   // re-read soon, from L2
                else if (!DIAM) st_stream(q, acc);                             // never re-read
            } else if (last) {
                if (!DIAM) st_stream(q, acc);                                  // level 0: nobody's tail
            } else {
                *q = acc;
            }
            if constexpr (DIAM) mx = max(mx, fmax_of(acc));
        }
        if (j + 1 < nseg) {   // segment j done here; segment j + 1 needs segment j + 1 - lag everywhere
            __syncthreads();
            if (threadIdx.x == 0) {
                asm volatile("red.release.gpu.global.add.u32 [%0], 1;" ::"l"(&p.wave_done[j]) : "memory");
                // lag 1: a grid barrier on segment j; relaxed spin (an acquire load per
                // poll would drop the L1 lines of the CTAs still working on this SM), then
                // one acquire fence
                const uint32_t w = j + 1 >= p.seg_lag ? j + 1 - p.seg_lag : j;
                if (j + 1 >= p.seg_lag && ld_flag(&p.wave_done[w]) < target) {
                    uint32_t ns = 32;
                    const uint64_t t0 = globaltimer_ns();
                    while (ld_flag(&p.wave_done[w]) < target) {
                        __nanosleep(ns);
                        ns = min(ns * 2, 256u);
                        if ((*(volatile uint32_t*)p.err & 2u) || globaltimer_ns() - t0 > 4000000000ull) {
                            atomicOr(p.err, 2u);   // watchdog: report, never hang
                            break;
                        }
                    }
                }
                asm volatile("fence.acq_rel.gpu;" ::: "memory");
            }
            __syncthreads();
        }
        vb = ve;
    }
    if constexpr (DIAM) {
        __shared__ uint32_t wmax[SWEEP_THREADS / 32];
        mx = __reduce_max_sync(0xFFFFFFFFu, mx);
        if ((threadIdx.x & 31) == 0) wmax[threadIdx.x >> 5] = mx;
        __syncthreads();
        if (threadIdx.x < 32) {
            uint32_t w = threadIdx.x < SWEEP_THREADS / 32 ? wmax[threadIdx.x] : 0u;
            w = __reduce_max_sync(0xFFFFFFFFu, w);
            if (threadIdx.x == 0 && w) atomicMax(diam, w);
        }
    }
}

bool seg_batch() {   // PHAST_SEG_BATCH (default 0: measured slower, fewer CTAs per SM)
    const char* e = std::getenv("PHAST_SEG_BATCH");
    return e && std::atoi(e) != 0;
}

template <int K, bool DIAM>
int seg_occupancy() {
    int b = 0;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, seg_batch() ? (const void*)sweep_seg_kernel<K, DIAM, true>
                                                                      : (const void*)sweep_seg_kernel<K, DIAM, false>,
                                                      SWEEP_THREADS, 0) !=
        cudaSuccess) {
        cudaGetLastError();
        return 1;
    }
    return b > 0 ? b : 1;
}

// ------------------------------------------------------------------ a3+a4 pipelined gather (variant 3)
// CTA chunks on the wavefront layout with a one-chunk lookahead: while chunk c is
// reduced from shared memory, the tail rows of the CTA's next chunk are already in
// flight into the other shared-memory stage (cp.async.cg, 16 B per lane, no register
// staging).  A chunk's dependencies are at least two iterations back (plan lag 2),
// so its gathers can be issued one iteration early.  Two CTA barriers per chunk.
constexpr uint32_t PIPE_STAGE_BYTES = 16384;   // tail rows of one chunk


template <int K>
struct PipeGeom {
    static constexpr uint32_t G = K / 4;                          // lanes (16 B each) per row
    static constexpr uint32_t AMAX = PIPE_STAGE_BYTES / (K * 4);  // staged arcs per chunk
    static constexpr uint32_t VPP = SWEEP_THREADS / G;
    static constexpr uint32_t CV = (VPP * 4 < AMAX / 2 ? VPP * 4 : AMAX / 2) < VPP ? VPP
                                   : (VPP * 4 < AMAX / 2 ? VPP * 4 : AMAX / 2);
};

template <int K, bool DIAM>
__global__ void __launch_bounds__(SWEEP_THREADS, 4) sweep_pipe_kernel(const uint32_t* __restrict__ first,
                                                                      const uint2* __restrict__ arcs,
                                                                      uint32_t* __restrict__ d,
                                                                      const uint32_t* __restrict__ flags,
                                                                      const uint32_t* __restrict__ tail_bits,
                                                                      SweepPlan p, uint32_t epoch,
                                                                      uint32_t* __restrict__ diam) {
    static_assert(K >= 4 && K % 4 == 0, "pipelined sweep needs 16-byte rows");
    using Geo = PipeGeom<K>;
    constexpr uint32_t G = Geo::G, AMAX = Geo::AMAX, VPP = Geo::VPP, CV = Geo::CV;
    extern __shared__ __align__(16) uint8_t pipe_smem[];
    uint4* rows = reinterpret_cast<uint4*>(pipe_smem);                                  // [2][AMAX*G]
    uint2* sarc = reinterpret_cast<uint2*>(pipe_smem + 2 * PIPE_STAGE_BYTES);           // [2][AMAX]
    uint32_t* sfirst = reinterpret_cast<uint32_t*>(sarc + 2 * AMAX);                   // [2][CV+1]
    __shared__ uint4 sinfo[3];   // chunk descriptors, indexed by iteration % 3 (thread 0 runs <1 iteration ahead)
    const uint32_t grid = gridDim.x;
    const uint32_t gl = threadIdx.x % G, grp = threadIdx.x / G;
    uint32_t mx = 0;

    // warp 0, non-blocking: are the chunks (of other CTAs) holding the tails of chunk c
    // complete?  A lookahead must never block: the CTA still owes its current chunk.
    // m, dl: the chunk's meta and this lane's first dependency id, loaded one iteration
    // ahead (so only the completion flags are read here)
    auto deps_done = [&](const uint4& m, uint32_t dl) {
        const uint32_t lane = threadIdx.x & 31, dend = m.w & 0x7FFFFFFFu;
        bool ok = (m.w >> 31) == 0u;                  // depends on this CTA's current chunk: not yet
        if (ok && m.z + lane < dend) ok = ld_acquire_gpu(&p.done[dl]) >= epoch;
        for (uint32_t i = m.z + lane + 32; ok && i < dend; i += 32)
            ok = ld_acquire_gpu(&p.done[__ldg(&p.wdeps[i])]) >= epoch;
        return __all_sync(0xFFFFFFFFu, ok);
    };
    // warp 0, blocking: acquire the completion flags of the tails' chunks of chunk c
    auto wait_dep = [&](uint32_t c) {
        const uint4 m = __ldg(&p.wmeta[c]);
        const uint32_t lane = threadIdx.x & 31, dend = m.w & 0x7FFFFFFFu;
        for (uint32_t i = m.z + lane; i < dend; i += 32) {
            const uint32_t x = __ldg(&p.wdeps[i]);
            if (ld_acquire_gpu(&p.done[x]) < epoch) {
                uint32_t ns = 32;
                const uint64_t t0 = globaltimer_ns();
                while (ld_acquire_gpu(&p.done[x]) < epoch) {
                    __nanosleep(ns);
                    ns = min(ns * 2, 256u);
                    if ((*(volatile uint32_t*)p.err & 2u) || globaltimer_ns() - t0 > 4000000000ull) {
                        atomicOr(p.err, 2u);   // watchdog: report, never hang
                        break;
                    }
                }
            }
        }
        __syncwarp();
    };
    __shared__ uint32_t s_ready[2];   // stage b's gathers were issued as a lookahead
    // all threads: offsets and arcs of the chunk described by sinfo[b] into stage b
    auto stage = [&](uint32_t b, uint32_t si) {
        const uint4 in = sinfo[si];
        for (uint32_t i = threadIdx.x; i <= in.y - in.x; i += SWEEP_THREADS) sfirst[b * (CV + 1) + i] = __ldg(&first[in.x + i]);
        if (in.w - in.z <= AMAX)
            for (uint32_t i = threadIdx.x; i < in.w - in.z; i += SWEEP_THREADS) sarc[b * AMAX + i] = __ldg(&arcs[in.z + i]);
    };
    // all threads: 16-byte cp.async of every tail row slice of stage b's chunk
    auto gather = [&](uint32_t b, uint32_t si) {
        const uint4 in = sinfo[si];
        const uint32_t na = in.w - in.z;
        if (na <= AMAX) {
            for (uint32_t i = threadIdx.x; i < na * G; i += SWEEP_THREADS) {
                const uint32_t a = i / G, part = i % G;
                const uint32_t t = sarc[b * AMAX + a].x;
                cp_async16(&rows[(size_t)b * AMAX * G + i], reinterpret_cast<const uint4*>(d + (size_t)t * K) + part);
            }
        }
        cp_async_commit();
    };

    uint32_t c = blockIdx.x;
    if (c < p.nchunks) {
        if (threadIdx.x == 0) sinfo[0] = __ldg(&p.pinfo[c]);
        __syncthreads();
        stage(0, 0);
        if (threadIdx.x < 32) wait_dep(c);
        if (threadIdx.x == 0) s_ready[0] = 1;
        __syncthreads();
        gather(0, 0);
    }
    uint4 nxt = make_uint4(0, 0, 0, 0);
    if (threadIdx.x == 0 && c + grid < p.nchunks) nxt = __ldg(&p.pinfo[c + grid]);
    uint4 wm = make_uint4(0, 0, 0, 0);   // warp 0: meta + first dependency of the next chunk
    uint32_t wd = 0;
    if (threadIdx.x < 32 && c + grid < p.nchunks) {
        wm = __ldg(&p.wmeta[c + grid]);
        if (wm.z + threadIdx.x < (wm.w & 0x7FFFFFFFu)) wd = __ldg(&p.wdeps[wm.z + threadIdx.x]);
    }
    uint32_t it = 0;
    for (; c < p.nchunks; c += grid, it++) {
        const uint32_t b = it & 1u;
        const uint32_t si = it % 3u, sn = (it + 1) % 3u;
        const uint32_t cn = c + grid;
        if (threadIdx.x == 0 && cn < p.nchunks) {
            sinfo[sn] = nxt;
            if (cn + grid < p.nchunks) nxt = __ldg(&p.pinfo[cn + grid]);   // one more iteration ahead
        }
        __syncthreads();                                                       // [A]
        if (threadIdx.x == 0 && it > 0)                                        // chunk c-grid fully written
            st_release_gpu(&p.done[c - grid], epoch);                          // (release, cumulative over the CTA)
        if (!s_ready[b]) {                               // no lookahead for c: wait (blocking) and gather now
            if (threadIdx.x < 32) wait_dep(c);
            __syncthreads();
            gather(b, si);
        }
        if (cn < p.nchunks) stage(b ^ 1u, sn);
        if (threadIdx.x < 32) {
            const bool ok = cn < p.nchunks && deps_done(wm, wd);
            if (threadIdx.x == 0) s_ready[b ^ 1u] = ok ? 1u : 0u;
            if (cn + grid < p.nchunks) {                                       // prefetch for the next lookahead
                wm = __ldg(&p.wmeta[cn + grid]);
                if (wm.z + threadIdx.x < (wm.w & 0x7FFFFFFFu)) wd = __ldg(&p.wdeps[wm.z + threadIdx.x]);
            }
        }
        cp_async_wait_all();                                                   // my slices of chunk c
        __syncthreads();                                                       // [B]
        if (cn < p.nchunks && s_ready[b ^ 1u]) gather(b ^ 1u, sn);             // lookahead: chunk cn in flight
        const uint4 in = sinfo[si];
        const bool staged = in.w - in.z <= AMAX;
        const uint32_t* fb = sfirst + b * (CV + 1);
        for (uint32_t base = in.x; base < in.y; base += VPP) {
            const uint32_t v = base + grp;
            if (v >= in.y) break;
            uint4 acc = make_uint4(INF, INF, INF, INF);
            if ((__ldg(&flags[v >> 5]) >> (v & 31)) & 1u)
                acc = __ldcg(reinterpret_cast<const uint4*>(d + (size_t)v * K) + gl);
            const uint32_t e0 = fb[v - in.x], e1 = fb[v - in.x + 1];
            if (staged) {
                for (uint32_t e = e0; e < e1; e++) {
                    const uint32_t a = e - in.z;
                    acc = relax(acc, rows[(size_t)b * AMAX * G + a * G + gl], sarc[b * AMAX + a].y);
                }
            } else {
                for (uint32_t e = e0; e < e1; e++) {
                    const uint2 a = __ldg(&arcs[e]);
                    acc = relax(acc, __ldcg(reinterpret_cast<const uint4*>(d + (size_t)a.x * K) + gl), a.y);
                }
            }
            const bool is_tail = (__ldg(&tail_bits[v >> 5]) >> (v & 31)) & 1u;
            if (!DIAM || is_tail) {
                uint4* q = reinterpret_cast<uint4*>(d + (size_t)v * K) + gl;
                if (is_tail) *q = acc; else st_stream(q, acc);
            }
            if constexpr (DIAM) mx = max(mx, fmax_of(acc));
        }
    }
    __syncthreads();
    if (threadIdx.x == 0 && it > 0) st_release_gpu(&p.done[c - grid], epoch);
    cp_async_wait_all();
    if constexpr (DIAM) {
        __shared__ uint32_t wmax[SWEEP_THREADS / 32];
        mx = __reduce_max_sync(0xFFFFFFFFu, mx);
        if ((threadIdx.x & 31) == 0) wmax[threadIdx.x >> 5] = mx;
        __syncthreads();
        if (threadIdx.x < 32) {
            uint32_t w = threadIdx.x < SWEEP_THREADS / 32 ? wmax[threadIdx.x] : 0u;
            w = __reduce_max_sync(0xFFFFFFFFu, w);
            if (threadIdx.x == 0 && w) atomicMax(diam, w);
        }
    }
}

template <int K>
size_t pipe_smem_bytes() {
    using Geo = PipeGeom<K>;
    return 2 * PIPE_STAGE_BYTES + 2 * Geo::AMAX * sizeof(uint2) + 2 * (Geo::CV + 1) * sizeof(uint32_t);
}

template <int K, bool DIAM>
int pipe_occupancy() {
    if constexpr (K < 4) {
        return 0;
    } else {
        static bool attr = false;
        if (!attr) {
            if (cudaFuncSetAttribute(sweep_pipe_kernel<K, DIAM>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                     (int)pipe_smem_bytes<K>()) != cudaSuccess) {
                cudaGetLastError();
                return 0;
            }
            attr = true;
        }
        int b = 0;
        if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, sweep_pipe_kernel<K, DIAM>, SWEEP_THREADS,
                                                          pipe_smem_bytes<K>()) != cudaSuccess) {
            cudaGetLastError();
            return 0;
        }
        return b;
    }
}

template <int K, bool DIAM, bool STAGE>
int persistent_occupancy() {
    int b = 0;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, sweep_persistent_kernel<K, DIAM, STAGE>, SWEEP_THREADS,
                                                      0) != cudaSuccess) {
        cudaGetLastError();
        return 1;
    }
    return b > 0 ? b : 1;
}

template <int K, bool STAGE>
cudaError_t persistent_k2(const DevImage& g, const SweepPlan& p, uint32_t epoch, uint32_t* dist, uint32_t* diam,
                          cudaStream_t st) {
    if (diam)
        sweep_persistent_kernel<K, true, STAGE><<<p.grid, SWEEP_THREADS, 0, st>>>(
            g.dn_first, g.dn_arc, dist, g.flags, g.tail_bits, p, epoch, diam);
    else
        sweep_persistent_kernel<K, false, STAGE><<<p.grid, SWEEP_THREADS, 0, st>>>(
            g.dn_first, g.dn_arc, dist, g.flags, g.tail_bits, p, epoch, nullptr);
    g_launches++;
    return cudaGetLastError();
}

template <int K>
cudaError_t persistent_k(const DevImage& g, const SweepPlan& p, uint32_t epoch, uint32_t* dist, uint32_t* diam,
                         cudaStream_t st) {
    if constexpr (K >= 4) {
        if (p.variant == 3) {
            const size_t smem = pipe_smem_bytes<K>();
            if (diam)
                sweep_pipe_kernel<K, true><<<p.grid, SWEEP_THREADS, smem, st>>>(g.dn_first, g.dn_arc, dist, g.flags,
                                                                                 g.tail_bits, p, epoch, diam);
            else
                sweep_pipe_kernel<K, false><<<p.grid, SWEEP_THREADS, smem, st>>>(g.dn_first, g.dn_arc, dist, g.flags,
                                                                                  g.tail_bits, p, epoch, nullptr);
            g_launches++;
            return cudaGetLastError();
        }
    }
    if (p.variant == 6) {
        const bool b = seg_batch();
        if (diam)
            (b ? sweep_seg_kernel<K, true, true> : sweep_seg_kernel<K, true, false>)<<<p.grid, SWEEP_THREADS, 0, st>>>(
                g.dn_first, g.dn_arc, dist, g.flags, g.tail_bits, p, epoch, diam);
        else
            (b ? sweep_seg_kernel<K, false, true> : sweep_seg_kernel<K, false, false>)<<<p.grid, SWEEP_THREADS, 0, st>>>(
                g.dn_first, g.dn_arc, dist, g.flags, g.tail_bits, p, epoch, nullptr);
        g_launches++;
        return cudaGetLastError();
    }
    if (p.variant == 5) {
        if (diam)
            sweep_wave_kernel<K, true><<<p.grid, SWEEP_THREADS, 0, st>>>(g.dn_first, g.dn_arc, dist, g.flags,
                                                                         g.tail_bits, p, epoch, diam);
        else
            sweep_wave_kernel<K, false><<<p.grid, SWEEP_THREADS, 0, st>>>(g.dn_first, g.dn_arc, dist, g.flags,
                                                                          g.tail_bits, p, epoch, nullptr);
        g_launches++;
        return cudaGetLastError();
    }
    if (p.variant == 4) {
        if (diam)
            sweep_wpipe_kernel<K, true><<<p.grid, SWEEP_THREADS, 0, st>>>(g.dn_first, g.dn_arc, dist, g.flags,
                                                                          g.tail_bits, p, epoch, diam);
        else
            sweep_wpipe_kernel<K, false><<<p.grid, SWEEP_THREADS, 0, st>>>(g.dn_first, g.dn_arc, dist, g.flags,
                                                                           g.tail_bits, p, epoch, nullptr);
        g_launches++;
        return cudaGetLastError();
    }
    if (p.variant == 2) {
        if (diam)
            sweep_warp_kernel<K, true><<<p.grid, SWEEP_THREADS, 0, st>>>(g.dn_first, g.dn_arc, dist, g.flags,
                                                                         g.tail_bits, p, epoch, diam);
        else
            sweep_warp_kernel<K, false><<<p.grid, SWEEP_THREADS, 0, st>>>(g.dn_first, g.dn_arc, dist, g.flags,
                                                                          g.tail_bits, p, epoch, nullptr);
        g_launches++;
        return cudaGetLastError();
    }
    return p.variant == 1 ? persistent_k2<K, true>(g, p, epoch, dist, diam, st)
                          : persistent_k2<K, false>(g, p, epoch, dist, diam, st);
}

cudaError_t upward_launch(const DevImage& g, const Sources& src, uint32_t k, uint32_t slot, uint32_t vtop,
                          cudaStream_t st) {
    static bool attr = false;
    size_t smem = 5 * (size_t)g.smem_cap * sizeof(uint32_t);
    if (!attr) {
        cudaError_t e = cudaFuncSetAttribute(upward_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                             (int)(5 * UP_SMEM_CAP * sizeof(uint32_t)));
        if (e != cudaSuccess) return e;
        attr = true;
    }
    upward_kernel<<<k, UP_THREADS, smem, st>>>(g, src, slot, vtop);
    g_launches++;
    return cudaGetLastError();
}

template <int K>
cudaError_t seed_rows_k(const DevImage& g, uint32_t k, uint32_t slot, uint32_t* dist, cudaStream_t st) {
    seed_rows_kernel<K><<<k, 256, 0, st>>>(g, slot, dist);
    g_launches++;
    return cudaGetLastError();
}

__global__ void max_reduce_kernel(const uint32_t* __restrict__ in, uint32_t count, uint32_t* out) {
    uint32_t mx = 0;
    for (uint32_t i = threadIdx.x; i < count; i += blockDim.x) mx = max(mx, in[i]);
    __shared__ uint32_t w[32];
    mx = __reduce_max_sync(0xFFFFFFFFu, mx);
    if ((threadIdx.x & 31) == 0) w[threadIdx.x >> 5] = mx;
    __syncthreads();
    if (threadIdx.x < 32) {
        uint32_t x = threadIdx.x < blockDim.x / 32 ? w[threadIdx.x] : 0u;
        x = __reduce_max_sync(0xFFFFFFFFu, x);
        if (threadIdx.x == 0) *out = x;
    }
}

}  // namespace

// ------------------------------------------------------------------ a3 + a4: top levels in one CTA
// The top of the hierarchy has many tiny levels (C1: 73 levels for 10 k vertices;
// C3: the top 46 levels hold 59 k of 18 M vertices).  One launch per level
// (§VI "The CPU starts, for each level i, a kernel on the GPU") costs
// ~4 us of launch + drain per level however small it is, so the levels whose rows
// fit in shared memory run in ONE CTA instead:
//  - the rows of [0, V) (the top levels: internal ids ascend as levels descend) live
//    in shared memory for the whole launch and are written back once;
//  - warp 0 is a producer: its 32 lanes stream every chunk's offsets and arcs
//    (contiguous per level, §IV-A) into a ring of `stages` shared-memory
//    stages with 16-byte cp.async, arriving on the stage's mbarrier, as far ahead as
//    the ring allows (DESIGN.md §6 lists the fills measured slower: TMA from one
//    lane, every thread's share, TMA after an L2 prefetch);
//  - 31 consumer warps relax one chunk at a time from shared memory
//    (§III "if d(v) > d(u)+l(u,v), we set d(v) = d(u)+l(u,v)") and meet
//    at a named barrier after it, which orders the levels (Lemma 4.1: every tail is
//    in an earlier chunk) and frees the ring stage.
// Two initialisations:
//  - top mode (fused = 0): rows = seeded label if visited, else INF (PAPER.md:16
//    §IV-C); the upward searches and the seeding ran before;
//  - fused mode (fused = 1, V = n, the whole graph): rows = INF except d_i(s_i) = 0,
//    and the chunks [0, split) are a PULL sweep of G-up in ascending level order
//    (in-arcs of A-up by head): afterwards every row holds the exact G-up distance
//    from its source, INF where G-up does not reach -- the result of the upward CH
//    search run to exhaustion (§III "it runs Dijkstra s algorithm from s
//    in G, stopping when the priority queue becomes empty"; reading R9), for every
//    vertex at once.  The chunks [split, nchunks) are then the downward sweep.  One
//    launch per query: no upward kernel, no seeding, no visited bits.
constexpr int TOP_THREADS = 1024, TOP_CONS = TOP_THREADS - 32;
// chunk geometry (per plan, TopArgs::big): small 256 vertices / 1 024 arcs (9 280-byte
// stages), big 1 024 / 4 096 (36 928-byte stages) when the rows leave room for 4 big
// stages: fewer, larger chunks = fewer barriers on the long levels of small-k queries
constexpr uint32_t TOP_VCH = 256, TOP_ECH = 1024, TOP_VCH_BIG = 1024, TOP_ECH_BIG = 4096;
__host__ __device__ constexpr uint32_t top_off_buf(bool big) { return (big ? TOP_VCH_BIG : TOP_VCH) + 8; }
__host__ __device__ constexpr size_t top_stage_bytes(bool big) {   // {descriptor, offsets, arcs}
    return 16 + top_off_buf(big) * 4 + ((big ? TOP_ECH_BIG : TOP_ECH) + 2) * 8;
}
constexpr size_t TOP_STAGE_BYTES = top_stage_bytes(false);
constexpr uint32_t TOP_MAX_STAGES = 24, TOP_MIN_STAGES = 4;
constexpr size_t TOP_SMEM_MAX = 227 * 1024;

constexpr uint32_t TOP_HEAVY = 8;   // in-arcs above which a warp relaxes the vertex (k <= 4)
constexpr uint32_t TOP_VMASK = 0x7FFFFFFFu;   // chunk vend; bit 31: the chunk has a vertex with > TOP_HEAVY in-arcs
__device__ __forceinline__ uint32_t warp_min(uint32_t a) { return __reduce_min_sync(0xFFFFFFFFu, a); }
__device__ __forceinline__ uint2 warp_min(uint2 a) { return make_uint2(warp_min(a.x), warp_min(a.y)); }
__device__ __forceinline__ uint4 warp_min(uint4 a) {
    return make_uint4(warp_min(a.x), warp_min(a.y), warp_min(a.z), warp_min(a.w));
}

__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}

template <int K, bool DIAM>
__global__ void __launch_bounds__(TOP_THREADS, 1) sweep_top_kernel(TopArgs A, Sources src, uint32_t* __restrict__ d,
                                                                   const uint32_t* __restrict__ flags,
                                                                   uint32_t* __restrict__ diam) {
    using T = typename RowT<K>::T;
    constexpr uint32_t W = RowT<K>::W;
    constexpr uint32_t G = K / W;   // lanes per vertex
    extern __shared__ __align__(16) unsigned char top_smem[];
    const uint32_t V = A.V, S = A.stages;
    T* srow = reinterpret_cast<T*>(top_smem);
    const size_t lab = ((size_t)V * G * sizeof(T) + 15) & ~(size_t)15;
    unsigned char* ring = top_smem + lab;                                   // [S] {offsets, arcs}
    const size_t SB = top_stage_bytes(A.big);
    const uint32_t OFFB = top_off_buf(A.big);
    uint64_t* full = reinterpret_cast<uint64_t*>(ring + (size_t)S * SB);
    uint64_t* empty = full + S;
    const uint32_t tid = threadIdx.x;
    if (tid == 0) {
        for (uint32_t s = 0; s < S; s++) {
            mbar_init(&full[s], 32);   // one cp.async arrival per producer lane
            mbar_init(&empty[s], 1);
        }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    const T* dr = reinterpret_cast<const T*>(d);
    if (A.fused) {   // every row INF, then d_i(s_i) = 0
        for (uint32_t i = tid; i < V * G; i += TOP_THREADS) srow[i] = inf_row<T>();
        __syncthreads();
        if (tid < K) reinterpret_cast<uint32_t*>(srow)[(size_t)src.s[tid] * K + tid] = 0u;
    } else {         // a2 (implicit init): seeded label if visited, else INF
        for (uint32_t i = tid; i < V * G; i += TOP_THREADS) {
            const uint32_t v = i / G;
            srow[i] = ((__ldg(&flags[v >> 5]) >> (v & 31)) & 1u) ? dr[i] : inf_row<T>();
        }
    }
    __syncthreads();
    uint32_t mx = 0;
    if (tid < 32) {   // producer warp: all 32 lanes copy (cp.async, 16 B each), then arrive
        // (measured: 1-D bulk copies (TMA) of these small blocks issue only every
        // ~600-2000 cycles from one SM, slower than the consumers; 16-byte cp.async
        // from 32 lanes keeps the ring ahead)
        // descriptors: each lane holds one of the current 32 and one of the next 32
        // (loaded a batch ahead), so the issue loop never waits on a global load
        const uint32_t lane = tid;
        uint4 cur = make_uint4(0, 0, 0, 0), nxt = make_uint4(0, 0, 0, 0);
        if (lane < A.nchunks) cur = __ldg(&A.chunks[lane]);
        if (32 + lane < A.nchunks) nxt = __ldg(&A.chunks[32 + lane]);
        uint32_t s = 0, ph = 0;   // stage and its use count parity
        for (uint32_t c = 0; c < A.nchunks; c++) {
            if ((c & 31) == 0 && c) {
                cur = nxt;
                if (c + 32 + lane < A.nchunks) nxt = __ldg(&A.chunks[c + 32 + lane]);
            }
            uint4 ch;   // {vbeg, vend | heavy bit, ebeg = first[vbeg], eend = first[vend]}
            ch.x = __shfl_sync(0xFFFFFFFFu, cur.x, c & 31);
            ch.y = __shfl_sync(0xFFFFFFFFu, cur.y, c & 31);
            ch.z = __shfl_sync(0xFFFFFFFFu, cur.z, c & 31);
            ch.w = __shfl_sync(0xFFFFFFFFu, cur.w, c & 31);
            if (c >= S) mbar_wait(&empty[s], ph ^ 1u);   // the stage's previous chunk consumed
            if (A.dbg && lane == 0) A.dbg[4 * c + 3] = clock64();
            const bool up = c < A.split;
            const uint32_t f0 = ch.x & ~3u, nf4 = ((ch.y & TOP_VMASK) + 1 - f0 + 3) / 4;   // 16-byte units
            const uint32_t a0 = ch.z & ~1u, na2 = (ch.w - a0 + 1) / 2;
            unsigned char* st = ring + (size_t)s * SB;
            const uint4* gf = reinterpret_cast<const uint4*>((up ? A.first[0] : A.first[1]) + f0);
            const uint4* ga = reinterpret_cast<const uint4*>((up ? A.arcs[0] : A.arcs[1]) + a0);
            for (uint32_t u = lane; u < 1 + nf4 + na2; u += 32) {
                if (u == 0) cp_async16(st, A.chunks + c);   // the consumers read the descriptor here
                else if (u <= nf4) cp_async16(st + 16 * u, gf + (u - 1));
                else cp_async16(st + 16 + OFFB * 4 + 16 * (u - 1 - nf4), ga + (u - 1 - nf4));
            }
            asm volatile("cp.async.mbarrier.arrive.noinc.shared::cta.b64 [%0];" ::"r"(smem_u32(&full[s])) : "memory");
            if (++s == S) { s = 0; ph ^= 1u; }
        }
    } else {
        const uint32_t ct = tid - 32;
        uint32_t s = 0, ph = 0;
        for (uint32_t c = 0; c < A.nchunks; c++) {
            if (A.dbg && ct == 0) A.dbg[4 * c] = clock64();
            mbar_wait(&full[s], ph);
            if (A.dbg && ct == 0) A.dbg[4 * c + 1] = clock64();
            const unsigned char* st = ring + (size_t)s * SB;
            const uint4 ch = *reinterpret_cast<const uint4*>(st);
            const uint32_t f0 = ch.x & ~3u, a0 = ch.z & ~1u;
            const uint32_t* sf = reinterpret_cast<const uint32_t*>(st + 16);
            const uint2* sa = reinterpret_cast<const uint2*>(st + 16 + OFFB * 4);
            const uint32_t vend = ch.y & TOP_VMASK;
            const bool heavy = G == 1 && (ch.y & ~TOP_VMASK);   // host: some vertex has > TOP_HEAVY in-arcs
            const uint32_t total = (vend - ch.x) * G;
            for (uint32_t t = ct; t < total; t += TOP_CONS) {
                const uint32_t v = ch.x + t / G, lane = t % G;
                const uint32_t e0 = sf[v - f0], e1 = sf[v + 1 - f0];
                if (heavy && e1 - e0 > TOP_HEAVY) continue;   // a warp takes it below
                T acc = srow[v * G + lane];
                // four arcs at a time: their loads (then their rows' loads) are
                // independent, so a vertex costs two shared-memory round trips per
                // four arcs instead of two per arc
                for (uint32_t e = e0; e < e1; e += 4) {
                    uint2 a[4];
                    T x[4];
#pragma unroll
                    for (int r = 0; r < 4; r++) a[r] = e + r < e1 ? sa[e + r - a0] : make_uint2(0u, INF);
#pragma unroll
                    for (int r = 0; r < 4; r++) x[r] = srow[a[r].x * G + lane];   // row 0 for padding (len INF)
#pragma unroll
                    for (int r = 0; r < 4; r++) acc = relax(acc, x[r], a[r].y);
                }
                srow[v * G + lane] = acc;
            }
            if (heavy) {
                // vertices with many in-arcs (the top of G-up: every lower neighbour is
                // an in-arc) would serialise a level on one thread: one warp each, the
                // lanes striding over the arcs, then a warp min
                const uint32_t wid = ct >> 5, wl = ct & 31, nv = vend - ch.x;
                for (uint32_t i = wid; i < nv; i += TOP_CONS / 32) {
                    const uint32_t v = ch.x + i;
                    const uint32_t e0 = sf[v - f0], e1 = sf[v + 1 - f0];
                    if (e1 - e0 <= TOP_HEAVY) continue;   // warp-uniform
                    T acc = wl == 0 ? srow[v] : inf_row<T>();
                    for (uint32_t e = e0 + wl; e < e1; e += 128) {   // four arcs per lane in flight
                        uint2 a[4];
                        T x[4];
#pragma unroll
                        for (int r = 0; r < 4; r++) a[r] = e + 32 * r < e1 ? sa[e + 32 * r - a0] : make_uint2(0u, INF);
#pragma unroll
                        for (int r = 0; r < 4; r++) x[r] = srow[a[r].x];
#pragma unroll
                        for (int r = 0; r < 4; r++) acc = relax(acc, x[r], a[r].y);
                    }
                    acc = warp_min(acc);
                    if (wl == 0) srow[v] = acc;
                }
            }
            if (A.dbg && ct == 0) A.dbg[4 * c + 2] = clock64();
            asm volatile("bar.sync 1, %0;" ::"n"(TOP_CONS) : "memory");   // chunk done: next level may read it
            if (ct == 0) mbar_arrive(&empty[s]);                          // ring stage free
            if (++s == S) { s = 0; ph ^= 1u; }
        }
    }
    __syncthreads();
    T* dw = reinterpret_cast<T*>(d);
    for (uint32_t i = tid; i < V * G; i += TOP_THREADS) {   // final rows (a5: the fused max over them)
        dw[i] = srow[i];
        if constexpr (DIAM) mx = max(mx, fmax_of(srow[i]));
    }
    if constexpr (DIAM) {
        mx = __reduce_max_sync(0xFFFFFFFFu, mx);
        if ((tid & 31) == 0 && mx) atomicMax(diam, mx);
    }
}

size_t top_ring_min() { return TOP_MIN_STAGES * TOP_STAGE_BYTES + 2 * TOP_MIN_STAGES * sizeof(uint64_t); }
size_t top_label_budget() { return TOP_SMEM_MAX - top_ring_min() - 16; }
uint32_t top_chunk_vertices(bool big) { return big ? TOP_VCH_BIG : TOP_VCH; }
uint32_t top_chunk_arcs(bool big) { return big ? TOP_ECH_BIG : TOP_ECH; }
bool top_big_fits(uint32_t k, uint32_t V) {   // rows + 4 big stages within shared memory
    const size_t lab = ((size_t)V * k * 4 + 15) & ~(size_t)15;
    return lab + 4 * (top_stage_bytes(true) + 16) <= TOP_SMEM_MAX;
}
uint32_t top_heavy_arcs() { return TOP_HEAVY; }

template <int K>
cudaError_t top_k(TopArgs A, const Sources& src, uint32_t* dist, const uint32_t* flags, uint32_t* diam,
                  cudaStream_t st) {
    const size_t lab = ((size_t)A.V * K * 4 + 15) & ~(size_t)15;
    if (lab > top_label_budget()) return cudaErrorInvalidValue;
    const size_t SB = top_stage_bytes(A.big);
    A.stages = (uint32_t)std::min<size_t>(TOP_MAX_STAGES, (TOP_SMEM_MAX - lab) / (SB + 16));
    if (const char* e = std::getenv("PHAST_TOP_STAGES"))   // experiment knob: a shallower ring
        A.stages = std::max<uint32_t>(2, std::min<uint32_t>(A.stages, (uint32_t)std::atoi(e)));
    const size_t smem = lab + A.stages * (SB + 16);
    static bool attr_set[2] = {false, false};
    auto kern = diam ? sweep_top_kernel<K, true> : sweep_top_kernel<K, false>;
    if (!attr_set[diam ? 1 : 0]) {
        cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)TOP_SMEM_MAX);
        if (e != cudaSuccess) return e;
        attr_set[diam ? 1 : 0] = true;
    }
    static unsigned long long* dbg = nullptr;
    const char* dpath = std::getenv("PHAST_TOP_DEBUG");
    if (dpath && !dbg) cudaMalloc(&dbg, (size_t)A.nchunks * 32);
    if (dpath) A.dbg = dbg;
    kern<<<1, TOP_THREADS, smem, st>>>(A, src, dist, flags, diam);
    g_launches++;
    if (dpath) {   // diagnostics only: dump the stamps of this launch
        std::vector<unsigned long long> hbuf((size_t)A.nchunks * 4);
        cudaStreamSynchronize(st);
        cudaMemcpy(hbuf.data(), dbg, hbuf.size() * 8, cudaMemcpyDeviceToHost);
        if (FILE* f = std::fopen(dpath, "wb")) { std::fwrite(hbuf.data(), 8, hbuf.size(), f); std::fclose(f); }
    }
    return cudaGetLastError();
}

// ------------------------------------------------------------------ a3 + a4: mid levels in one cluster
// After the shared-memory top levels come levels of a few thousand vertices: too big
// for one SM, too small to amortise a launch (~4-5 us each with programmatic
// dependent launch).  They run in ONE launch of a thread-block cluster (C CTAs of
// 1 024 threads on C SMs): each level is a grid-stride pass over (vertex, 16-byte
// lane) items exactly like sweep_kernel's ELL path, and the level boundary
// (§VI: a kernel boundary in the paper) is a hardware cluster barrier
// with release/acquire semantics (barrier.cluster.arrive.release / wait.acquire),
// which orders the rows written by every CTA of the cluster before the next level
// reads them (Lemma 4.1: tails are in earlier levels).  Tail rows are read with
// ld.global.cg (L2): another SM wrote them in this launch.  The next level's first
// record is prefetched into L2 before the barrier (static data).
constexpr int CL_THREADS = 1024;

__device__ __forceinline__ void cluster_sync_acqrel() {
    asm volatile("barrier.cluster.arrive.release.aligned;\nbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}

template <int K, bool DIAM>
__global__ void __launch_bounds__(CL_THREADS, 1) sweep_cluster_kernel(const uint4* __restrict__ rec,
                                                                      const uint2* __restrict__ ovf,
                                                                      uint32_t* __restrict__ d,
                                                                      const uint32_t* __restrict__ flags,
                                                                      const uint32_t* __restrict__ seg,
                                                                      uint32_t nseg, uint32_t* __restrict__ diam) {
    using T = typename RowT<K>::T;
    constexpr uint32_t G = K / RowT<K>::W;   // lanes per vertex
    asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
    const uint32_t stride = gridDim.x * CL_THREADS;
    const uint32_t t0 = blockIdx.x * CL_THREADS + threadIdx.x;
    if (t0 < (__ldg(&seg[1]) - __ldg(&seg[0])) * G) asm volatile("prefetch.global.L2 [%0];" ::"l"(rec + __ldg(&seg[0]) + t0 / G));
    asm volatile("griddepcontrol.wait;" ::: "memory");   // the previous launch (top levels) complete
    uint32_t mx = 0;
    uint32_t vb = __ldg(&seg[0]);
    for (uint32_t j = 0; j < nseg; j++) {
        const uint32_t ve = __ldg(&seg[j + 1]);
        const uint32_t total = (ve - vb) * G;
        for (uint32_t t = t0; t < total; t += stride) {
            const uint32_t v = vb + t / G, lane = t % G;
            T acc = inf_row<T>();
            if ((__ldg(&flags[v >> 5]) >> (v & 31)) & 1u)   // visited by an upward search
                acc = __ldcg(reinterpret_cast<const T*>(d + (size_t)v * K) + lane);
            const uint4 r = __ldg(&rec[v]);
            T x0 = inf_row<T>(), x1 = inf_row<T>();
            if (r.y != INF) x0 = __ldcg(reinterpret_cast<const T*>(d + (size_t)r.x * K) + lane);
            if (r.w != INF) x1 = __ldcg(reinterpret_cast<const T*>(d + (size_t)r.z * K) + lane);
            acc = relax(relax(acc, x0, r.y), x1, r.w);
            if (r.w == INF && r.z != INF) {   // more than two in-arcs
                const uint2* o = ovf + r.z;
                const uint32_t cnt = __ldg(&o->x);
                for (uint32_t i = 1; i <= cnt; i++) {
                    const uint2 a = __ldg(&o[i]);
                    acc = relax(acc, __ldcg(reinterpret_cast<const T*>(d + (size_t)a.x * K) + lane), a.y);
                }
            }
            reinterpret_cast<T*>(d + (size_t)v * K)[lane] = acc;
            if constexpr (DIAM) mx = max(mx, fmax_of(acc));
        }
        if (j + 1 < nseg) {
            const uint32_t nb = __ldg(&seg[j + 2]);
            if (t0 < (nb - ve) * G) asm volatile("prefetch.global.L2 [%0];" ::"l"(rec + ve + t0 / G));
            cluster_sync_acqrel();   // level j final everywhere in the cluster
        }
        vb = ve;
    }
    if constexpr (DIAM) {
        mx = __reduce_max_sync(0xFFFFFFFFu, mx);
        if ((threadIdx.x & 31) == 0 && mx) atomicMax(diam, mx);
    }
}

// PHAST_CL_SIZE: CTAs per cluster (16 non-portable, 8 portable); default 0 = off:
// measured slower than per-level launches (C3 k=64 sweep 2.06-2.12 vs 2.03 ms; C2
// k=16 0.160 vs 0.132 ms; C2D 0.357 vs 0.377 ms, r42): a level inside the cluster
// costs about what a programmatic-dependent launch costs, on 16 SMs instead of 148.
int cluster_size() {
    const char* e = std::getenv("PHAST_CL_SIZE");
    int c = e ? std::atoi(e) : 0;
    return c <= 0 ? 0 : c > 16 ? 16 : c;
}

template <int K>
cudaError_t cluster_k(const DevImage& g, const uint32_t* seg, uint32_t nseg, uint32_t* dist, uint32_t* diam,
                      cudaStream_t st) {
    const int C = cluster_size();
    auto kern = diam ? sweep_cluster_kernel<K, true> : sweep_cluster_kernel<K, false>;
    static bool attr_set[2] = {false, false};
    if (!attr_set[diam ? 1 : 0]) {
        cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
        if (e != cudaSuccess) return e;
        attr_set[diam ? 1 : 0] = true;
    }
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3((unsigned)C);
    cfg.blockDim = dim3(CL_THREADS);
    cfg.stream = st;
    cudaLaunchAttribute attr[2];
    attr[0].id = cudaLaunchAttributeClusterDimension;
    attr[0].val.clusterDim.x = (unsigned)C;
    attr[0].val.clusterDim.y = 1;
    attr[0].val.clusterDim.z = 1;
    attr[1].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr[1].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 2;
    cudaError_t e = cudaLaunchKernelEx(&cfg, kern, g.dn_rec, g.dn_ovf, dist, (const uint32_t*)g.flags, seg, nseg, diam);
    if (e != cudaSuccess && C > 8) {   // a 16-CTA cluster may not fit this GPU's GPCs: portable size 8
        cudaGetLastError();
        cfg.gridDim = dim3(8u);
        attr[0].val.clusterDim.x = 8u;
        e = cudaLaunchKernelEx(&cfg, kern, g.dn_rec, g.dn_ovf, dist, (const uint32_t*)g.flags, seg, nseg, diam);
    }
    g_launches++;
    return e;
}

#define PHAST_K_SWITCH(k, CALL)      \
    switch (k) {                     \
        case 1: return CALL(1);      \
        case 2: return CALL(2);      \
        case 4: return CALL(4);      \
        case 8: return CALL(8);      \
        case 16: return CALL(16);    \
        case 32: return CALL(32);    \
        case 64: return CALL(64);    \
        default: return cudaErrorInvalidValue; \
    }

cudaError_t launch_upward(const DevImage& g, const Sources& src, uint32_t k, uint32_t slot, uint32_t vtop,
                          cudaStream_t st) {
    return upward_launch(g, src, k, slot, vtop, st);
}

cudaError_t launch_seed(const DevImage& g, uint32_t k, uint32_t slot, uint32_t* dist, cudaStream_t st) {
#define CALL_SR(K) seed_rows_k<K>(g, k, slot, dist, st)
    cudaError_t e = [&]() -> cudaError_t { PHAST_K_SWITCH(k, CALL_SR) }();
#undef CALL_SR
    if (e != cudaSuccess) return e;
    scatter_kernel<<<k, 256, 0, st>>>(g, slot, k, dist);
    g_launches++;
    return cudaGetLastError();
}

cudaError_t launch_sweep_level(const DevImage& g, uint32_t k, uint32_t vbeg, uint32_t vend, uint32_t* dist,
                               uint32_t* diam, bool store, bool last_level, bool by_tail, cudaStream_t st) {
#define CALL_SW(K) sweep_k<K>(g, vbeg, vend, dist, diam, store, last_level, by_tail, st)
    PHAST_K_SWITCH(k, CALL_SW)
#undef CALL_SW
}

void sweep_pipe_geometry(uint32_t k, uint32_t* cap_vertices, uint32_t* cap_arcs) {
    switch (k) {
        case 4: *cap_vertices = PipeGeom<4>::CV; *cap_arcs = PipeGeom<4>::AMAX; return;
        case 8: *cap_vertices = PipeGeom<8>::CV; *cap_arcs = PipeGeom<8>::AMAX; return;
        case 16: *cap_vertices = PipeGeom<16>::CV; *cap_arcs = PipeGeom<16>::AMAX; return;
        case 32: *cap_vertices = PipeGeom<32>::CV; *cap_arcs = PipeGeom<32>::AMAX; return;
        case 64: *cap_vertices = PipeGeom<64>::CV; *cap_arcs = PipeGeom<64>::AMAX; return;
        default: *cap_vertices = 0; *cap_arcs = 0; return;
    }
}

uint32_t sweep_wpipe_chunk_vertices(uint32_t k) {
    switch (k) {
        case 1: return WpGeom<1>::CAP;
        case 2: return WpGeom<2>::CAP;
        case 4: return WpGeom<4>::CAP;
        case 8: return WpGeom<8>::CAP;
        case 16: return WpGeom<16>::CAP;
        case 32: return WpGeom<32>::CAP;
        default: return WpGeom<64>::CAP;
    }
}

uint32_t sweep_wave_chunk_vertices(uint32_t k) {
    switch (k) {
        case 1: return WaveGeom<1>::U;
        case 2: return WaveGeom<2>::U;
        case 4: return WaveGeom<4>::U;
        case 8: return WaveGeom<8>::U;
        case 16: return WaveGeom<16>::U;
        case 32: return WaveGeom<32>::U;
        default: return WaveGeom<64>::U;
    }
}
uint32_t sweep_wave_chunk_arcs() { return WAVE_ACAP - 2; }
uint32_t sweep_wave_subcounters() { return WAVE_SUB; }

uint32_t sweep_warp_chunk_vertices(uint32_t k) { return (32 / (k >= 4 ? k / 4 : 1)) * WARP_PASSES; }

uint32_t sweep_pass_vertices(uint32_t k) { return SWEEP_THREADS / (k >= 4 ? k / 4 : 1); }

uint32_t sweep_chunk_vertices(uint32_t k) {
    uint32_t G = k >= 4 ? k / 4 : 1;
    return (SWEEP_THREADS / G) * CHUNK_PASSES;
}

int sweep_blocks_per_sm(uint32_t k, bool diam, uint32_t variant) {
#define OCC(K)                                                                                               \
    (variant == 6 ? (diam ? seg_occupancy<K, true>() : seg_occupancy<K, false>()) :                           \
     variant == 5 ? (diam ? wave_occupancy<K, true>() : wave_occupancy<K, false>()) :                         \
     variant == 4 ? (diam ? wpipe_occupancy<K, true>() : wpipe_occupancy<K, false>()) :                       \
     variant == 3 ? (diam ? pipe_occupancy<K, true>() : pipe_occupancy<K, false>()) :                         \
     variant == 2 ? (diam ? warp_occupancy<K, true>() : warp_occupancy<K, false>()) :                         \
     variant == 1 ? (diam ? persistent_occupancy<K, true, true>() : persistent_occupancy<K, false, true>())   \
                  : (diam ? persistent_occupancy<K, true, false>() : persistent_occupancy<K, false, false>()))
    switch (k) {
        case 1: return OCC(1);
        case 2: return OCC(2);
        case 4: return OCC(4);
        case 8: return OCC(8);
        case 16: return OCC(16);
        case 32: return OCC(32);
        case 64: return OCC(64);
        default: return 1;
    }
#undef OCC
}

cudaError_t launch_sweep_persistent(const DevImage& g, const SweepPlan& p, uint32_t epoch, uint32_t* dist,
                                    uint32_t* diam, cudaStream_t st) {
#define CALL_PS(K) persistent_k<K>(g, p, epoch, dist, diam, st)
    PHAST_K_SWITCH(p.k, CALL_PS)
#undef CALL_PS
}

cudaError_t launch_parents(const uint32_t* in_first, const uint2* in_arc, uint32_t n, const Sources& src,
                           uint32_t k, const uint32_t* dist, uint32_t* parent, cudaStream_t st) {
#define CALL_PA(K) parents_k<K>(in_first, in_arc, n, src, dist, parent, st)
    PHAST_K_SWITCH(k, CALL_PA)
#undef CALL_PA
}

cudaError_t launch_sweep_top(const TopArgs& A, uint32_t k, const Sources& src, uint32_t* dist,
                             const uint32_t* flags, uint32_t* diam, cudaStream_t st) {
#define CALL_TOP(K) top_k<K>(A, src, dist, flags, diam, st)
    PHAST_K_SWITCH(k, CALL_TOP)
#undef CALL_TOP
}

cudaError_t launch_sweep_cluster(const DevImage& g, uint32_t k, const uint32_t* seg, uint32_t nseg, uint32_t* dist,
                                 uint32_t* diam, cudaStream_t st) {
#define CALL_CL(K) cluster_k<K>(g, seg, nseg, dist, diam, st)
    PHAST_K_SWITCH(k, CALL_CL)
#undef CALL_CL
}
uint32_t cluster_threads() { return cluster_size() > 0 ? (uint32_t)cluster_size() * CL_THREADS : 0u; }

cudaError_t launch_clear_flags(const DevImage& g, uint32_t k, uint32_t slot, cudaStream_t st) {
    clear_flags_kernel<<<k, 256, 0, st>>>(g, slot);
    g_launches++;
    return cudaGetLastError();
}

cudaError_t launch_max_reduce(const uint32_t* in, uint32_t count, uint32_t* out, cudaStream_t st) {
    max_reduce_kernel<<<1, 1024, 0, st>>>(in, count, out);
    g_launches++;
    return cudaGetLastError();
}

}  // namespace phast

// ------------------------------------------------------------------ NEXT-3 betweenness
// Exact (partial) betweenness on top of k finished trees (§VII-B "c_B(v) =
// sum_{s != v != t} sigma_st(v)/sigma_st").  Rows are [n][k]
// like the labels.  With lengths > 0 the tight arcs d(u) + l = d(w) of a tree form a
// DAG, and sigma (path counts) and delta (Brandes' dependencies) are the unique
// solutions of
//   sigma(v) = [v = s] + sum_{tight (u, v)} sigma(u)
//   delta(v) = sum_{tight (v, w)} sigma(v) / sigma(w) * (1 + delta(w)).
// Both kernels are one in-place (chaotic) relaxation pass over every (vertex, tree);
// the host repeats a pass until one changes nothing, which is then the fixpoint.  Each
// value is a fixed function of its inputs summed in a fixed arc order, so the result
// does not depend on the schedule.  sigma is an integer in fp64 (exact below 2^53).
// The in-place reads race benignly with writes of other threads (aligned 8-byte
// stores); plain loads (not __ldg) so a pass sees writes of earlier passes.
namespace phast {
namespace {
__device__ __forceinline__ bool tight(uint32_t du, uint32_t dv, uint32_t l) {
    return du <= dv && dv - du == l;   // du + l == dv without 32-bit overflow
}
}  // namespace

// Schedule (not part of the method): Kahn's topological order of each tree's tight DAG.
// An item t = v*k + i is computed ONCE, when all its inputs are final: cnt[t] counts the
// item's unfinished inputs (forward: tight in-arcs; backward: tight out-arcs); a pass
// computes the items of its queue and, for each dependent whose count drops to zero,
// appends it to the next queue.  Passes = hop depth of the tight DAG + 1; each pass
// touches only its frontier.  Queue sizes rotate over three counters: pass p reads
// qs[p%3], appends with qs[(p+1)%3] and zeroes qs[(p+2)%3].
__device__ __forceinline__ void bc_push(uint32_t t, uint32_t* q, uint32_t* qs, bool& pushed) {
    q[atomicAdd(qs, 1u)] = t;
    pushed = true;
}

// cnt[t] = number of inputs of item t; items with none start the first queue
__global__ void __launch_bounds__(256) bc_count_kernel(BcGraph G, const uint32_t* __restrict__ d, uint32_t n,
                                                       uint32_t k, int backward, uint32_t* cnt, uint32_t* q,
                                                       uint32_t* qs) {
    const uint64_t total = (uint64_t)n * k;
    bool pushed = false;
    for (uint64_t t = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; t < total;
         t += (uint64_t)gridDim.x * blockDim.x) {
        const uint32_t v = (uint32_t)(t / k), i = (uint32_t)(t % k);
        const uint32_t dv = __ldg(&d[t]);
        if (dv == INF) continue;
        uint32_t c = 0;
        if (!backward) {
            const uint32_t e1 = __ldg(&G.in_first[v + 1]);
            for (uint32_t e = __ldg(&G.in_first[v]); e < e1; e++) {
                const uint2 a = __ldg(&G.in_arc[e]);
                c += tight(__ldg(&d[(size_t)a.x * k + i]), dv, a.y);
            }
        } else {
            const uint32_t e1 = __ldg(&G.out_first[v + 1]);
            for (uint32_t e = __ldg(&G.out_first[v]); e < e1; e++) {
                const uint2 a = __ldg(&G.out_arc[e]);
                const uint32_t dw = __ldg(&d[(size_t)a.x * k + i]);
                c += dw != INF && tight(dv, dw, a.y);
            }
        }
        cnt[t] = c;
        if (c == 0) bc_push((uint32_t)t, q, qs, pushed);
    }
    (void)pushed;
}

// forward pass: sigma(v) = [v = s] + sum over tight (u, v) of sigma(u).  With lengths > 0
// the source is the only finite item without a tight in-arc, so [v = s] is "no tight
// in-arc" (no source list in the parameters: the passes are graph-captured once per call)
__global__ void __launch_bounds__(256) bc_sigma_kernel(BcGraph G, const uint32_t* __restrict__ d, double* sigma,
                                                       uint32_t k, BcQueue Q, uint32_t* changed) {
    const uint32_t size = *Q.qs_in;
    if (blockIdx.x == 0 && threadIdx.x == 0) *Q.qs_clr = 0;
    bool pushed = false;
    for (uint32_t x = blockIdx.x * blockDim.x + threadIdx.x; x < size; x += gridDim.x * blockDim.x) {
        const uint32_t t = Q.q_in[x];
        const uint32_t v = t / k, i = t % k;
        const uint32_t dv = __ldg(&d[t]);
        double acc = 0.0;
        bool any = false;
        const uint32_t e1 = __ldg(&G.in_first[v + 1]);
        for (uint32_t e = __ldg(&G.in_first[v]); e < e1; e++) {
            const uint2 a = __ldg(&G.in_arc[e]);
            const size_t u = (size_t)a.x * k + i;
            if (tight(__ldg(&d[u]), dv, a.y)) {
                acc += sigma[u];
                any = true;
            }
        }
        sigma[t] = any ? acc : 1.0;
        const uint32_t f1 = __ldg(&G.out_first[v + 1]);
        for (uint32_t e = __ldg(&G.out_first[v]); e < f1; e++) {
            const uint2 a = __ldg(&G.out_arc[e]);
            const uint32_t w = a.x * k + i;
            const uint32_t dw = __ldg(&d[w]);
            if (dw != INF && tight(dv, dw, a.y) && atomicSub(&Q.cnt[w], 1u) == 1u) bc_push(w, Q.q_out, Q.qs_out, pushed);
        }
    }
    if (__syncthreads_or(pushed) && threadIdx.x == 0) *changed = 1;
}

// backward pass; mode 0: delta(v) = sum over tight (v, w) of sigma(v)/sigma(w) (1 + delta(w));
// mode 1 (reach): height h(v) = max over tight (v, w) of l + h(w), stored as uint32 in
// `val` (l + h(w) <= d(w) + h(w) - d(v) is at most the largest finite label: no wrap)
__global__ void __launch_bounds__(256) bc_back_kernel(BcGraph G, const uint32_t* __restrict__ d,
                                                      const double* __restrict__ sigma, void* val, uint32_t k,
                                                      int mode, BcQueue Q, uint32_t* changed) {
    const uint32_t size = *Q.qs_in;
    if (blockIdx.x == 0 && threadIdx.x == 0) *Q.qs_clr = 0;
    bool pushed = false;
    double* delta = static_cast<double*>(val);
    uint32_t* hgt = static_cast<uint32_t*>(val);
    for (uint32_t x = blockIdx.x * blockDim.x + threadIdx.x; x < size; x += gridDim.x * blockDim.x) {
        const uint32_t t = Q.q_in[x];
        const uint32_t v = t / k, i = t % k;
        const uint32_t dv = __ldg(&d[t]);
        const uint32_t e1 = __ldg(&G.out_first[v + 1]);
        if (mode == 0) {
            const double sv = __ldg(&sigma[t]);
            double acc = 0.0;
            for (uint32_t e = __ldg(&G.out_first[v]); e < e1; e++) {
                const uint2 a = __ldg(&G.out_arc[e]);
                const size_t w = (size_t)a.x * k + i;
                const uint32_t dw = __ldg(&d[w]);
                if (dw != INF && tight(dv, dw, a.y)) acc += sv / __ldg(&sigma[w]) * (1.0 + delta[w]);
            }
            delta[t] = acc;
        } else {
            uint32_t acc = 0;
            for (uint32_t e = __ldg(&G.out_first[v]); e < e1; e++) {
                const uint2 a = __ldg(&G.out_arc[e]);
                const size_t w = (size_t)a.x * k + i;
                const uint32_t dw = __ldg(&d[w]);
                if (dw != INF && tight(dv, dw, a.y)) acc = max(acc, a.y + hgt[w]);
            }
            hgt[t] = acc;
        }
        const uint32_t f1 = __ldg(&G.in_first[v + 1]);
        for (uint32_t e = __ldg(&G.in_first[v]); e < f1; e++) {
            const uint2 a = __ldg(&G.in_arc[e]);
            const uint32_t u = a.x * k + i;
            if (tight(__ldg(&d[u]), dv, a.y) && atomicSub(&Q.cnt[u], 1u) == 1u) bc_push(u, Q.q_out, Q.qs_out, pushed);
        }
    }
    if (__syncthreads_or(pushed) && threadIdx.x == 0) *changed = 1;
}

// Persistent form of the Kahn passes: ONE cooperative launch runs every pass of one
// direction, moving to the next pass on a grid-wide barrier (no launch or host check
// per pass).  Values written in earlier passes by other SMs are read with ld.global.cg
// (L2, not the incoherent L1); the queue size of a pass is final at the barrier before
// it, so every thread sees the same size and leaves the loop together.
// mode 0: sigma (forward); 1: delta (backward); 2: height (backward).
__global__ void __launch_bounds__(256) bc_kahn_persistent_kernel(BcGraph G, const uint32_t* __restrict__ d,
                                                                 double* sigma, void* val, uint32_t k, int mode,
                                                                 uint32_t* q0, uint32_t* q1, uint32_t* qs,
                                                                 uint32_t* cnt, uint32_t max_passes, uint32_t* err) {
    namespace cg = cooperative_groups;
    cg::grid_group grid = cg::this_grid();
    double* delta = static_cast<double*>(val);
    uint32_t* hgt = static_cast<uint32_t*>(val);
    const uint32_t gtid = blockIdx.x * blockDim.x + threadIdx.x, gthreads = gridDim.x * blockDim.x;
    for (uint32_t p = 0;; p++) {
        const uint32_t* q_in = (p & 1) ? q1 : q0;
        uint32_t* q_out = (p & 1) ? q0 : q1;
        uint32_t* qs_out = qs + (p + 1) % 3;
        const uint32_t size = __ldcg(qs + p % 3);
        if (size == 0) break;
        if (p >= max_passes) {   // cannot happen with lengths > 0
            if (gtid == 0) atomicOr(err, 2u);
            break;
        }
        if (gtid == 0) qs[(p + 2) % 3] = 0;
        for (uint32_t x = gtid; x < size; x += gthreads) {
            const uint32_t t = __ldcg(q_in + x);
            const uint32_t v = t / k, i = t % k;
            const uint32_t dv = __ldg(&d[t]);
            if (mode == 0) {
                double acc = 0.0;
                bool any = false;
                const uint32_t e1 = __ldg(&G.in_first[v + 1]);
                for (uint32_t e = __ldg(&G.in_first[v]); e < e1; e++) {
                    const uint2 a = __ldg(&G.in_arc[e]);
                    const size_t u = (size_t)a.x * k + i;
                    if (tight(__ldg(&d[u]), dv, a.y)) {
                        acc += __ldcg(sigma + u);
                        any = true;
                    }
                }
                sigma[t] = any ? acc : 1.0;
                const uint32_t f1 = __ldg(&G.out_first[v + 1]);
                for (uint32_t e = __ldg(&G.out_first[v]); e < f1; e++) {
                    const uint2 a = __ldg(&G.out_arc[e]);
                    const uint32_t w = a.x * k + i;
                    const uint32_t dw = __ldg(&d[w]);
                    if (dw != INF && tight(dv, dw, a.y) && atomicSub(&cnt[w], 1u) == 1u) q_out[atomicAdd(qs_out, 1u)] = w;
                }
            } else {
                const uint32_t e1 = __ldg(&G.out_first[v + 1]);
                if (mode == 1) {
                    const double sv = __ldg(&sigma[t]);
                    double acc = 0.0;
                    for (uint32_t e = __ldg(&G.out_first[v]); e < e1; e++) {
                        const uint2 a = __ldg(&G.out_arc[e]);
                        const size_t w = (size_t)a.x * k + i;
                        const uint32_t dw = __ldg(&d[w]);
                        if (dw != INF && tight(dv, dw, a.y)) acc += sv / __ldg(&sigma[w]) * (1.0 + __ldcg(delta + w));
                    }
                    delta[t] = acc;
                } else {
                    uint32_t acc = 0;
                    for (uint32_t e = __ldg(&G.out_first[v]); e < e1; e++) {
                        const uint2 a = __ldg(&G.out_arc[e]);
                        const size_t w = (size_t)a.x * k + i;
                        const uint32_t dw = __ldg(&d[w]);
                        if (dw != INF && tight(dv, dw, a.y)) acc = max(acc, a.y + __ldcg(hgt + w));
                    }
                    hgt[t] = acc;
                }
                const uint32_t f1 = __ldg(&G.in_first[v + 1]);
                for (uint32_t e = __ldg(&G.in_first[v]); e < f1; e++) {
                    const uint2 a = __ldg(&G.in_arc[e]);
                    const uint32_t u = a.x * k + i;
                    if (tight(__ldg(&d[u]), dv, a.y) && atomicSub(&cnt[u], 1u) == 1u) q_out[atomicAdd(qs_out, 1u)] = u;
                }
            }
        }
        grid.sync();
    }
}

// c_B(v) += sum over the first kv trees i (in order) with sources[i] != v of delta_i(v)
__global__ void __launch_bounds__(256) bc_accum_kernel(const double* __restrict__ delta, double* __restrict__ cb,
                                                       uint32_t n, uint32_t k, uint32_t kv, Sources src) {
    for (uint32_t v = blockIdx.x * blockDim.x + threadIdx.x; v < n; v += gridDim.x * blockDim.x) {
        double s = 0.0;
        for (uint32_t i = 0; i < kv; i++)
            if (src.s[i] != v) s += __ldg(&delta[(size_t)v * k + i]);
        cb[v] += s;
    }
}

// r(v) = max(r(v), max over the first kv trees of min(d_i(v), h_i(v)))
__global__ void __launch_bounds__(256) reach_accum_kernel(const uint32_t* __restrict__ d,
                                                          const uint32_t* __restrict__ hgt, uint32_t* __restrict__ r,
                                                          uint32_t n, uint32_t k, uint32_t kv) {
    for (uint32_t v = blockIdx.x * blockDim.x + threadIdx.x; v < n; v += gridDim.x * blockDim.x) {
        uint32_t m = r[v];
        for (uint32_t i = 0; i < kv; i++) {
            const uint32_t dv = __ldg(&d[(size_t)v * k + i]);
            if (dv != INF) m = max(m, min(dv, __ldg(&hgt[(size_t)v * k + i])));
        }
        r[v] = m;
    }
}

static unsigned bc_blocks(uint64_t items) {
    uint64_t b = (items + 255) / 256;
    return (unsigned)std::max<uint64_t>(1, std::min<uint64_t>(b, (uint64_t)num_sms() * 8));
}

cudaError_t launch_bc_count(const BcGraph& G, const uint32_t* d, uint32_t n, uint32_t k, int backward, uint32_t* cnt,
                            uint32_t* q, uint32_t* qs, cudaStream_t st) {
    bc_count_kernel<<<bc_blocks((uint64_t)n * k), 256, 0, st>>>(G, d, n, k, backward, cnt, q, qs);
    g_launches++;
    return cudaGetLastError();
}

// the passes touch only their queue: a small fixed grid (queue sizes are read on the device)
static unsigned bc_pass_blocks(uint64_t items) { return std::min<unsigned>(bc_blocks(items), (unsigned)num_sms() * 2); }

cudaError_t launch_bc_sigma(const BcGraph& G, const uint32_t* d, double* sigma, uint32_t n, uint32_t k,
                            const BcQueue& Q, uint32_t* changed, cudaStream_t st) {
    bc_sigma_kernel<<<bc_pass_blocks((uint64_t)n * k), 256, 0, st>>>(G, d, sigma, k, Q, changed);
    g_launches++;
    return cudaGetLastError();
}

cudaError_t launch_bc_back(const BcGraph& G, const uint32_t* d, const double* sigma, void* val, uint32_t n, uint32_t k,
                           int mode, const BcQueue& Q, uint32_t* changed, cudaStream_t st) {
    bc_back_kernel<<<bc_pass_blocks((uint64_t)n * k), 256, 0, st>>>(G, d, sigma, val, k, mode, Q, changed);
    g_launches++;
    return cudaGetLastError();
}

cudaError_t launch_bc_persistent(const BcGraph& G, const uint32_t* d, double* sigma, void* val, uint32_t k, int mode,
                                 uint32_t* q0, uint32_t* q1, uint32_t* qs, uint32_t* cnt, uint32_t max_passes,
                                 uint32_t* err, cudaStream_t st) {
    static int per_sm = -1;
    if (per_sm < 0) {
        int b = 0;
        if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, bc_kahn_persistent_kernel, 256, 0) != cudaSuccess) b = 0;
        per_sm = std::min(b, 2);
    }
    if (per_sm <= 0) return cudaErrorCooperativeLaunchTooLarge;
    void* args[] = {(void*)&G, (void*)&d, (void*)&sigma, (void*)&val, (void*)&k, (void*)&mode, (void*)&q0,
                    (void*)&q1, (void*)&qs, (void*)&cnt, (void*)&max_passes, (void*)&err};
    cudaError_t e = cudaLaunchCooperativeKernel((const void*)bc_kahn_persistent_kernel, dim3(num_sms() * per_sm),
                                                dim3(256), args, 0, st);
    g_launches++;
    return e;
}

cudaError_t launch_reach_accum(const uint32_t* d, const uint32_t* hgt, uint32_t* r, uint32_t n, uint32_t k, uint32_t kv,
                               cudaStream_t st) {
    reach_accum_kernel<<<bc_blocks(n), 256, 0, st>>>(d, hgt, r, n, k, kv);
    g_launches++;
    return cudaGetLastError();
}

cudaError_t launch_bc_accum(const double* delta, double* cb, uint32_t n, uint32_t k, uint32_t kv, const Sources& src,
                            cudaStream_t st) {
    bc_accum_kernel<<<bc_blocks(n), 256, 0, st>>>(delta, cb, n, k, kv, src);
    g_launches++;
    return cudaGetLastError();
}

}  // namespace phast
