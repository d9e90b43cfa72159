// sweep.cu -- PHAST's hot path on sm_100a.
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
//                        16-byte label loads per lane.
// a5 diameter          : max over finite labels fused into the sweep (PAPER.md:20
//                        §VII-B "making each core keep track of the maximum label it
//                        encounters"); witness argmax.
// No tensor cores: the loop is an integer (min,+) gather with no reuse.
#include <algorithm>
#include <atomic>
#include <mutex>
#include <set>
#include <utility>

#include "device.cuh"
#include "kernels.h"

namespace phast {

static std::atomic<uint64_t> g_launches{0};
uint64_t launches() { return g_launches.load(); }
void add_launches(int64_t d) { g_launches += (uint64_t)d; }
void count_launch() { g_launches++; }

int num_sms() {
    static std::atomic<int> cache[64];
    int dev = 0;
    if (cudaGetDevice(&dev) != cudaSuccess) { cudaGetLastError(); return 148; }
    if (dev < 0 || dev >= 64) return 148;
    int s = cache[dev].load();
    if (!s) {
        if (cudaDeviceGetAttribute(&s, cudaDevAttrMultiProcessorCount, dev) != cudaSuccess || s <= 0) {
            cudaGetLastError();
            s = 148;
        }
        cache[dev] = s;
    }
    return s;
}

cudaError_t ensure_smem_attr(const void* kernel, int bytes) {
    static std::mutex mu;
    static std::set<std::pair<const void*, int>> done;   // (kernel, device)
    int dev = 0;
    cudaError_t e = cudaGetDevice(&dev);
    if (e != cudaSuccess) return e;
    std::lock_guard<std::mutex> lk(mu);
    if (done.count({kernel, dev})) return cudaSuccess;
    e = cudaFuncSetAttribute(kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, bytes);
    if (e == cudaSuccess) done.insert({kernel, dev});
    return e;
}

namespace {

constexpr uint32_t EMPTY = 0xFFFFFFFFu;
constexpr int UP_THREADS = 512;
constexpr uint32_t UP_SMEM_CAP = 4096;   // shared-memory table entries per source (max)

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
    uint32_t qn, nn, used, over, over_next, cnt;   // over_next: set during a wave, published between waves
};

// Returns the slot of w (inserting it), or EMPTY when the table is 3/4 full.
__device__ __forceinline__ uint32_t up_insert(const UpTable& t, uint32_t w, UpShared& c) {
    const uint32_t mask = t.cap - 1;
    uint32_t h = hash32(w) & mask;
    for (uint32_t probe = 0; probe < t.cap; probe++) {
        const uint32_t k = *((volatile uint32_t*)&t.keys[h]);
        if (k == w) return h;
        if (k == EMPTY) {
            if (atomicAdd(&c.used, 0u) * 4 >= t.cap * 3) return EMPTY;
            const uint32_t old = atomicCAS(&t.keys[h], EMPTY, w);
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
__device__ bool up_search(const uint32_t* __restrict__ up_first, const uint2* __restrict__ up_arc, uint32_t s,
                          UpTable t, UpShared& c, uint32_t vtop) {
    const uint32_t tid = threadIdx.x;
    for (uint32_t i = tid; i < t.cap; i += blockDim.x) { t.keys[i] = EMPTY; t.vals[i] = INF; t.inq[i] = 0; }
    __syncthreads();
    if (tid == 0) {
        const uint32_t h = hash32(s) & (t.cap - 1);
        t.keys[h] = s; t.vals[h] = 0; t.inq[h] = 1; t.qa[0] = h;
        c.qn = s >= vtop ? 1u : 0u; c.nn = 0; c.used = 1; c.over = 0; c.over_next = 0; c.cnt = 0;
    }
    __syncthreads();
    uint32_t* qa = t.qa;
    uint32_t* qb = t.qb;
    for (;;) {
        const uint32_t qn = c.qn;
        if (qn == 0 || c.over) break;
        for (uint32_t idx = tid; idx < qn; idx += blockDim.x) {
            const uint32_t slot = qa[idx];
            atomicExch(&t.inq[slot], 0u);
            __threadfence_block();
            const uint32_t v = t.keys[slot];
            const uint32_t dv = *((volatile uint32_t*)&t.vals[slot]);
            const uint32_t e1 = __ldg(&up_first[v + 1]);
            for (uint32_t e = __ldg(&up_first[v]); e < e1; e++) {
                const uint2 a = __ldg(&up_arc[e]);
                const uint32_t nd = sat_add(dv, a.y);
                if (nd == INF) continue;
                const uint32_t ws = up_insert(t, a.x, c);
                if (ws == EMPTY) { c.over_next = 1; break; }
                const uint32_t old = atomicMin(&t.vals[ws], nd);
                if (nd < old && a.x >= vtop) {
                    __threadfence_block();
                    if (atomicExch(&t.inq[ws], 1u) == 0u) qb[atomicAdd(&c.nn, 1u)] = ws;
                }
            }
        }
        __syncthreads();
        if (tid == 0) { c.qn = c.nn; c.nn = 0; c.over = c.over_next; }   // every thread reads these after the barrier
        uint32_t* tmp = qa; qa = qb; qb = tmp;
        __syncthreads();
    }
    const bool ok = !c.over;
    __syncthreads();
    return ok;
}

// a1: search only; the search space goes to the slot's seed buffers (the sweep of
// the previous batch may still be running: nothing here touches the visited bits or
// the label rows).
__global__ void __launch_bounds__(UP_THREADS) upward_kernel(DevImage g, Slot sl, Sources src, uint32_t vtop) {
    extern __shared__ uint32_t smem[];
    __shared__ UpShared c;
    const uint32_t i = blockIdx.x;
    const uint32_t s = src.s[i];
    const uint32_t sc = g.smem_cap;
    UpTable t{smem, smem + sc, smem + 2 * sc, smem + 3 * sc, smem + 4 * sc, sc};
    bool ok = up_search(g.up_first, g.up_arc, s, t, c, vtop);
    if (!ok) {   // global-memory fallback with the per-source capacity (the slot's own
                 // table set: searches of different slots may run at once)
        uint32_t* base = sl.gscratch + (size_t)i * g.seed_cap * 5;
        UpTable gt{base, base + g.seed_cap, base + 2 * (size_t)g.seed_cap, base + 3 * (size_t)g.seed_cap,
                   base + 4 * (size_t)g.seed_cap, g.seed_cap};
        t = gt;
        ok = up_search(g.up_first, g.up_arc, s, t, c, vtop);
        if (!ok) {
            if (threadIdx.x == 0) { atomicOr(g.err, 1u); sl.seed_cnt[i] = 0; }
            return;
        }
    }
    uint32_t* sv = sl.seed_v + (size_t)i * g.seed_cap;
    uint32_t* sd = sl.seed_d + (size_t)i * g.seed_cap;
    for (uint32_t e = threadIdx.x; e < t.cap; e += blockDim.x) {
        const uint32_t v = t.keys[e];
        if (v == EMPTY) continue;
        const uint32_t pos = atomicAdd(&c.cnt, 1u);
        sv[pos] = v;
        sd[pos] = t.vals[e];
    }
    __syncthreads();
    if (threadIdx.x == 0) sl.seed_cnt[i] = c.cnt;
}

// ------------------------------------------------------------------ a2 seeding
// phase 1: visited bits of the search space, and its rows reset to INF
template <int K>
__global__ void seed_rows_kernel(Slot sl, uint32_t seed_cap, uint32_t* __restrict__ dist) {
    const uint32_t i = blockIdx.x;
    const uint32_t cnt = sl.seed_cnt[i];
    const uint32_t* sv = sl.seed_v + (size_t)i * seed_cap;
    for (uint32_t j = threadIdx.x; j < cnt; j += blockDim.x) {
        const uint32_t v = sv[j];
        atomicOr(&sl.flags[v >> 5], 1u << (v & 31));
    }
    using T = typename RowT<K>::T;
    constexpr uint32_t G = K / RowT<K>::W;
    for (uint32_t j = threadIdx.x; j < cnt * G; j += blockDim.x)
        reinterpret_cast<T*>(dist + (size_t)sv[j / G] * K)[j % G] = inf_row<T>();
}

// phase 2 (after every reset of phase 1): the labels
__global__ void scatter_kernel(Slot sl, uint32_t seed_cap, uint32_t k, uint32_t* __restrict__ dist) {
    const uint32_t i = blockIdx.x;
    const uint32_t cnt = sl.seed_cnt[i];
    const uint32_t* sv = sl.seed_v + (size_t)i * seed_cap;
    const uint32_t* sd = sl.seed_d + (size_t)i * seed_cap;
    for (uint32_t j = threadIdx.x; j < cnt; j += blockDim.x) dist[(size_t)sv[j] * k + i] = sd[j];
}

__global__ void clear_flags_kernel(Slot sl, uint32_t seed_cap) {
    const uint32_t i = blockIdx.x;
    const uint32_t cnt = sl.seed_cnt[i];
    const uint32_t* sv = sl.seed_v + (size_t)i * seed_cap;
    for (uint32_t j = threadIdx.x; j < cnt; j += blockDim.x) sl.flags[sv[j] >> 5] = 0u;
}

// ------------------------------------------------------------------ a3 sweep
constexpr int SWEEP_THREADS = 256;

// One level [vbeg, vend) (§VI "The CPU starts, for each level i, a kernel on
// the GPU").  One (vertex, 16-byte lane) item per thread per grid-stride step; the
// grid fills every SM (8 CTAs of 256 threads), which keeps the most gathers in flight.
// Each vertex's first two in-arcs come from one 16-byte ELL-2 record (97 % of level-0
// and 92 % of level-1 vertices at C3 have at most two), so the tail-row gathers depend
// on ONE load; more in-arcs continue in the overflow list.  Launched with programmatic
// dependent launch: the next level's grid is launched while this one drains and blocks
// in griddepcontrol.wait until this grid's rows are visible; the graph is static, so
// the first record is prefetched into L2 before the wait.
// NOGATHER (probe A34, §VIII-B "it takes 153 ms to traverse the graph
// exactly as PHAST does, but storing at d(v) the sum of the lengths of all arcs into
// v"): identical traversal, with every tail row replaced by the arc's length.
// WIDE (levels where many vertices have 3-4 in-arcs): a second record with arcs 2-3 is
// loaded beside the first, so up to four gathers depend on one round trip.
template <int K, bool DIAM, bool STORE, bool STREAM, bool NOGATHER, bool WIDE>
__global__ void __launch_bounds__(SWEEP_THREADS, WIDE ? 6 : 8)   // WIDE: registers for four rows in flight
    sweep_kernel(const uint4* __restrict__ rec, const uint4* __restrict__ rec2, const uint2* __restrict__ ovf,
                 uint32_t* __restrict__ d, const uint32_t* __restrict__ flags, uint32_t vbeg, uint32_t vend,
                 uint32_t* __restrict__ diam) {
    using T = typename RowT<K>::T;
    constexpr uint32_t G = K / RowT<K>::W;   // lanes per vertex
    asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
    const uint32_t total = (vend - vbeg) * G;   // host: < 2^31 (sweep_launch splits longer levels)
    uint32_t t = blockIdx.x * SWEEP_THREADS + threadIdx.x;
    if (t < total) asm volatile("prefetch.global.L2 [%0];" ::"l"(rec + vbeg + t / G));
    asm volatile("griddepcontrol.wait;" ::: "memory");   // previous level complete and visible
    uint32_t mx = 0;
    for (; t < total; t += gridDim.x * SWEEP_THREADS) {
        const uint32_t v = vbeg + t / G;
        const uint32_t lane = t % G;
        T acc = inf_row<T>();
        if (visited(flags, v)) acc = __ldg(reinterpret_cast<const T*>(d + (size_t)v * K) + lane);
        const uint4 r = __ldg(&rec[v]);
        uint4 r2 = make_uint4(0u, INF, 0u, INF);
        if constexpr (WIDE) r2 = __ldg(&rec2[v]);
        const bool more = WIDE ? (r2.w == INF && r2.z != INF) : (r.w == INF && r.z != INF);   // overflow list
        const uint32_t oi = WIDE ? r2.z : r.z;
        if constexpr (NOGATHER) {
            acc = splat<T>(sat_add(sat_add(min(r.y, 0xFFFFFFFEu), r.w == INF ? 0u : r.w),
                                   sat_add(r2.y == INF ? 0u : r2.y, (r2.w == INF || !WIDE) ? 0u : r2.w)));
        } else {
            // a missing arc has len INF: relaxing an INF row by it changes nothing
            T x0 = inf_row<T>(), x1 = inf_row<T>(), x2 = inf_row<T>(), x3 = inf_row<T>();
            if (r.y != INF) x0 = __ldg(reinterpret_cast<const T*>(d + (size_t)r.x * K) + lane);
            if (r.w != INF) x1 = __ldg(reinterpret_cast<const T*>(d + (size_t)r.z * K) + lane);
            if constexpr (WIDE) {
                if (r2.y != INF) x2 = __ldg(reinterpret_cast<const T*>(d + (size_t)r2.x * K) + lane);
                if (r2.w != INF) x3 = __ldg(reinterpret_cast<const T*>(d + (size_t)r2.z * K) + lane);
            }
            acc = relax(relax(acc, x0, r.y), x1, r.w);
            if constexpr (WIDE) acc = relax(relax(acc, x2, r2.y), x3, r2.w);
        }
        if (more) {   // the rest in the overflow list
            const uint2* o = ovf + oi;
            const uint32_t cnt = __ldg(&o->x);
            for (uint32_t j = 1; j <= cnt; j++) {
                const uint2 a = __ldg(&o[j]);
                if constexpr (NOGATHER) acc = splat<T>(sat_add(fmax_of(acc), a.y));
                else acc = relax(acc, __ldg(reinterpret_cast<const T*>(d + (size_t)a.x * K) + lane), a.y);
            }
        }
        if constexpr (STORE) {
            T* p = reinterpret_cast<T*>(d + (size_t)v * K) + lane;
            if constexpr (STREAM) __stcs(p, acc); else *p = acc;
        }
        if constexpr (DIAM) mx = max(mx, fmax_of(acc));
    }
    if constexpr (DIAM) cta_max_to<SWEEP_THREADS>(mx, diam);
}

template <int K, bool DIAM, bool STORE, bool STREAM, bool NOGATHER, bool WIDE>
cudaError_t sweep_launch(const DevImage& g, const uint32_t* flags, uint32_t vbeg, uint32_t vend, uint32_t* dist,
                         uint32_t* diam, cudaStream_t st) {
    constexpr uint32_t G = K / RowT<K>::W;
    constexpr uint32_t VMAX = (1u << 31) / G;   // 32-bit item indices in the kernel
    if (vend - vbeg > VMAX) {                    // a level has no internal arcs: split it freely
        cudaError_t e = sweep_launch<K, DIAM, STORE, STREAM, NOGATHER, WIDE>(g, flags, vbeg, vbeg + VMAX, dist, diam, st);
        return e != cudaSuccess ? e
                                : sweep_launch<K, DIAM, STORE, STREAM, NOGATHER, WIDE>(g, flags, vbeg + VMAX, vend, dist,
                                                                                       diam, st);
    }
    const uint64_t total = (uint64_t)(vend - vbeg) * G;
    uint64_t blocks = (total + SWEEP_THREADS - 1) / SWEEP_THREADS;
    const uint64_t cap = (uint64_t)num_sms() * (WIDE ? 6 : 8);   // one full wave of resident CTAs (launch bounds)
    if (blocks > cap) blocks = cap;
    if (blocks == 0) return cudaSuccess;
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3((unsigned)blocks);
    cfg.blockDim = dim3(SWEEP_THREADS);
    cfg.dynamicSmemBytes = 0;
    cfg.stream = st;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    cudaError_t e = cudaLaunchKernelEx(&cfg, sweep_kernel<K, DIAM, STORE, STREAM, NOGATHER, WIDE>, g.dn_rec, g.dn_rec2,
                                       g.dn_ovf, dist, flags, vbeg, vend, diam);
    count_launch();
    return e;
}

template <int K, bool WIDE>
cudaError_t sweep_kw(const DevImage& g, const uint32_t* flags, uint32_t vbeg, uint32_t vend, uint32_t* dist,
                     uint32_t* diam, bool store, bool last, bool nogather, cudaStream_t st) {
    if (nogather) return sweep_launch<K, false, true, false, true, WIDE>(g, flags, vbeg, vend, dist, diam, st);
    if (diam) {
        if (!store) return sweep_launch<K, true, false, false, false, WIDE>(g, flags, vbeg, vend, dist, diam, st);
        return last ? sweep_launch<K, true, true, true, false, WIDE>(g, flags, vbeg, vend, dist, diam, st)
                    : sweep_launch<K, true, true, false, false, WIDE>(g, flags, vbeg, vend, dist, diam, st);
    }
    return last ? sweep_launch<K, false, true, true, false, WIDE>(g, flags, vbeg, vend, dist, diam, st)
                : sweep_launch<K, false, true, false, false, WIDE>(g, flags, vbeg, vend, dist, diam, st);
}

template <int K>
cudaError_t sweep_k(const DevImage& g, const uint32_t* flags, uint32_t vbeg, uint32_t vend, uint32_t* dist,
                    uint32_t* diam, bool store, bool last, bool nogather, bool wide, cudaStream_t st) {
    return wide ? sweep_kw<K, true>(g, flags, vbeg, vend, dist, diam, store, last, nogather, st)
                : sweep_kw<K, false>(g, flags, vbeg, vend, dist, diam, store, last, nogather, st);
}

// ------------------------------------------------------------------ a3 band sweep
// Band kernel variants (BandArgs::variant; schedule choices, same labels).  Measured
// on C3 (profiles/r2_band_variants.md), the product keeps the ablation of
// the three that matter:
//   bit 0 PF_REG : each thread loads the next item's record while it gathers the
//                  current item's tail rows (48 registers: 1280 threads per SM)
//   bit 2 L1     : tail rows read through the L1 (band_ld); 28-42 % L1 hits
//   bit 3 LPT2   : two 16-byte lanes per thread (U8; 64 registers, 1024 threads per SM):
//                  two loads in flight per tail row, the record / flag / address work
//                  amortised over 32 bytes of row
// 13 = all three (the default for k >= 32), 5 = PF_REG + L1 (k = 16), 0 = none (k < 16),
// 1, 4.  Measured slower and removed: four lanes per thread, L2 bulk prefetch of the
// next unit's records, two items per thread in flight, records chained across levels
// and units or prefetched across the level barrier, no barrier between units, 1536 /
// 2048 threads per SM with spills, cp.async-staged gathers, in-unit rows in shared memory.
template <int VAR>
constexpr int band_sm_threads_of() { return (VAR & 8) ? 1024 : (VAR & 1) ? 1280 : 1536; }

// The static inputs of one (vertex, lane) item of a band level: its ELL record(s) and
// its visited-bit word.
struct BandRec {
    uint4 r, r2;
    uint32_t fl;
};
template <bool WIDE>
__device__ __forceinline__ BandRec band_rec(const uint4* __restrict__ rec, const uint4* __restrict__ rec2,
                                            const uint32_t* __restrict__ flags, uint32_t v) {
    BandRec b;
    b.r = __ldg(&rec[v]);
    b.r2 = make_uint4(0u, INF, 0u, INF);
    if constexpr (WIDE) b.r2 = __ldg(&rec2[v]);
    b.fl = __ldg(&flags[v >> 5]);
    return b;
}

// One (vertex, lane) item of a band level.  Tail rows are read with ld.global.cg: rows
// of the same work unit were written by this CTA earlier in this launch (visible after
// the level barrier; the L1 is bypassed), rows from above the band by earlier launches.
// Row loads of the band kernel: L1 = true reads through the L1 (plain ld.global: the
// PTX memory model makes rows written by this CTA before the level barrier visible;
// every row is written once per query and never read before its write in a launch, and
// the L1 is invalidated at launch boundaries), false bypasses it (ld.global.cg).
template <bool L1, class T>
__device__ __forceinline__ T band_ld(const T* p) {
    if constexpr (L1) return *p;
    else return __ldcg(p);
}

// Two 16-byte lanes per thread (variant bit 3, k >= 8; U8 in device.cuh): half the
// items, two loads in flight per tail row per thread, the per-item record / flag /
// address work amortised over 32 bytes of row.
template <bool L1>
__device__ __forceinline__ U8 band_ld(const U8* p) {
    const uint4* q = reinterpret_cast<const uint4*>(p);
    return U8{band_ld<L1>(q), band_ld<L1>(q + 1)};
}
__device__ __forceinline__ U8 ldcg_row(const U8* p) {
    const uint4* q = reinterpret_cast<const uint4*>(p);
    return U8{__ldcg(q), __ldcg(q + 1)};
}
template <class T> __device__ __forceinline__ T ldcg_row(const T* p) { return __ldcg(p); }
__device__ __forceinline__ void stcs_row(U8* p, U8 x) {
    uint4* q = reinterpret_cast<uint4*>(p);
    __stcs(q, x.a);
    __stcs(q + 1, x.b);
}
template <class T> __device__ __forceinline__ void stcs_row(T* p, T x) { __stcs(p, x); }
// lanes per thread: LPT = 1 (RowT) or 2 (U8, k >= 8)
template <int K, int LPT> struct BandLane { using T = typename RowT<K>::T; static constexpr uint32_t G = K / RowT<K>::W; };
template <int K> struct BandLane<K, 2> { using T = U8; static constexpr uint32_t G = K / 8; };

template <int K, bool WIDE, bool DIAM, bool L1 = false, int LPT2 = 1>
__device__ __forceinline__ void band_item(const BandRec& b, const uint2* __restrict__ ovf, uint32_t* __restrict__ d,
                                          uint32_t v, uint32_t lane, bool store, bool stream, uint32_t& mx) {
    using T = typename BandLane<K, LPT2>::T;
    const uint4 r = b.r, r2 = b.r2;
    T acc = inf_row<T>();
    // the seeded own row: never through the L1 (this item overwrites it)
    if ((b.fl >> (v & 31)) & 1u) acc = ldcg_row(reinterpret_cast<const T*>(d + (size_t)v * K) + lane);
    const bool more = WIDE ? (r2.w == INF && r2.z != INF) : (r.w == INF && r.z != INF);
    const uint32_t oi = WIDE ? r2.z : r.z;
    T x0 = inf_row<T>(), x1 = inf_row<T>(), x2 = inf_row<T>(), x3 = inf_row<T>();
    if (r.y != INF) x0 = band_ld<L1>(reinterpret_cast<const T*>(d + (size_t)r.x * K) + lane);
    if (r.w != INF) x1 = band_ld<L1>(reinterpret_cast<const T*>(d + (size_t)r.z * K) + lane);
    if constexpr (WIDE) {
        if (r2.y != INF) x2 = band_ld<L1>(reinterpret_cast<const T*>(d + (size_t)r2.x * K) + lane);
        if (r2.w != INF) x3 = band_ld<L1>(reinterpret_cast<const T*>(d + (size_t)r2.z * K) + lane);
    }
    acc = relax(relax(acc, x0, r.y), x1, r.w);
    if constexpr (WIDE) acc = relax(relax(acc, x2, r2.y), x3, r2.w);
    if (more) {
        const uint2* o = ovf + oi;
        const uint32_t cnt = __ldg(&o->x);
        for (uint32_t j = 1; j <= cnt; j++) {
            const uint2 a = __ldg(&o[j]);
            acc = relax(acc, band_ld<L1>(reinterpret_cast<const T*>(d + (size_t)a.x * K) + lane), a.y);
        }
    }
    if (store) {
        T* p = reinterpret_cast<T*>(d + (size_t)v * K) + lane;
        if (stream) stcs_row(p, acc); else *p = acc;
    }
    if constexpr (DIAM) mx = max(mx, fmax_of(acc));
}

// One unit level [vb, ve).  PF_REG: the next item's record is loaded before the
// current item's gathers.
template <int K, bool WIDE, bool DIAM, int THREADS, bool PF_REG, bool L1, int LPT2>
__device__ __forceinline__ void band_level(const uint4* __restrict__ rec, const uint4* __restrict__ rec2,
                                           const uint2* __restrict__ ovf, uint32_t* __restrict__ d,
                                           const uint32_t* __restrict__ flags, uint32_t vb, uint32_t ve, bool store,
                                           bool stream, uint32_t& mx) {
    constexpr uint32_t G = BandLane<K, LPT2>::G;
    const uint32_t total = (ve - vb) * G;
    uint32_t t = threadIdx.x;
    if constexpr (PF_REG) {
        if (t >= total) return;
        BandRec nx = band_rec<WIDE>(rec, rec2, flags, vb + t / G);
        for (;;) {
            const BandRec cur = nx;
            const uint32_t tn = t + THREADS;
            if (tn < total) nx = band_rec<WIDE>(rec, rec2, flags, vb + tn / G);
            band_item<K, WIDE, DIAM, L1, LPT2>(cur, ovf, d, vb + t / G, t % G, store, stream, mx);
            if (tn >= total) break;
            t = tn;
        }
    } else {
        for (; t < total; t += THREADS)
            band_item<K, WIDE, DIAM, L1, LPT2>(band_rec<WIDE>(rec, rec2, flags, vb + t / G), ovf, d, vb + t / G,
                                               t % G, store, stream, mx);
    }
}

// A band of levels in one launch (kernels.h BandArgs; layout.h Band).  Work units are
// dealt round-robin to a grid of one resident wave, so the units in flight at any time
// are neighbours in BFS order and share the rows they read from above the band.  The
// unit's level ranges go to shared memory once per unit (the next unit's are loaded
// into registers while this one is swept).
template <int K, bool DIAM, int THREADS, int VAR>
__global__ void __launch_bounds__(THREADS, band_sm_threads_of<VAR>() / THREADS)
    sweep_band_kernel(BandArgs a, const uint4* __restrict__ rec, const uint4* __restrict__ rec2,
                const uint2* __restrict__ ovf, uint32_t* __restrict__ d, const uint32_t* __restrict__ flags,
                uint32_t* __restrict__ diam) {
    static_assert(THREADS >= 32, "one warp at least");
    constexpr bool PF_REG = VAR & 1, L1 = VAR & 4;
    constexpr int LPT2 = ((VAR & 8) && K >= 8) ? 2 : 1;   // lanes per thread
    __shared__ uint32_t rng[2][32][2];   // [buffer][level][begin, end]
    asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
    asm volatile("griddepcontrol.wait;" ::: "memory");   // the levels above the band are complete and visible
    uint32_t mx = 0;
    const uint32_t U1 = a.U + 1, F = a.F, tid = threadIdx.x;
    uint32_t nb = 0, ne = 0;   // thread j < F: level j's range of the next unit
    uint32_t u = blockIdx.x;
    if (u < a.U && tid < F) { nb = __ldg(&a.off[tid * U1 + u]); ne = __ldg(&a.off[tid * U1 + u + 1]); }
    for (uint32_t buf = 0; u < a.U; u += gridDim.x, buf ^= 1u) {
        if (tid < F) { rng[buf][tid][0] = nb; rng[buf][tid][1] = ne; }
        __syncthreads();   // ranges visible; also orders this unit after the previous one
        const uint32_t un = u + gridDim.x;
        if (un < a.U && tid < F) { nb = __ldg(&a.off[tid * U1 + un]); ne = __ldg(&a.off[tid * U1 + un + 1]); }
        for (uint32_t j = 0; j < F; j++) {
            const uint32_t vb = rng[buf][j][0], ve = rng[buf][j][1];
            const bool last = j + 1 == F;
            const bool store = !last || a.store_last, stream = last && a.stream_last;
            if ((a.wide >> j) & 1u)
                band_level<K, true, DIAM, THREADS, PF_REG, L1, LPT2>(rec, rec2, ovf, d, flags, vb, ve, store, stream,
                                                                     mx);
            else
                band_level<K, false, DIAM, THREADS, PF_REG, L1, LPT2>(rec, rec2, ovf, d, flags, vb, ve, store, stream,
                                                                      mx);
            if (!last) __syncthreads();   // level j's rows are written before level j+1 reads them
        }
    }
    if constexpr (DIAM) cta_max_to<THREADS>(mx, diam);
}

// the band kernels use < 1 KB of shared memory: give the rest of the SM's 256 KB to the L1
cudaError_t prefer_l1(const void* kern) {
    static std::mutex mu;
    static std::set<std::pair<const void*, int>> done;
    int dev = 0;
    cudaError_t e = cudaGetDevice(&dev);
    if (e != cudaSuccess) return e;
    std::lock_guard<std::mutex> lk(mu);
    if (done.count({kern, dev})) return cudaSuccess;
    e = cudaFuncSetAttribute(kern, cudaFuncAttributePreferredSharedMemoryCarveout, 0);
    if (e == cudaSuccess) done.insert({kern, dev});
    return e;
}

template <int K, int THREADS, int VAR>
cudaError_t band_kt(const DevImage& g, const BandArgs& a, const uint32_t* flags, uint32_t* dist, uint32_t* diam,
                    cudaStream_t st) {
    if (VAR & 4) {
        cudaError_t e = prefer_l1(diam ? (const void*)sweep_band_kernel<K, true, THREADS, VAR>
                                       : (const void*)sweep_band_kernel<K, false, THREADS, VAR>);
        if (e != cudaSuccess) return e;
    }
    uint64_t blocks = std::min<uint64_t>(a.U, (uint64_t)num_sms() * (band_sm_threads_of<VAR>() / THREADS));
    if (blocks == 0 || a.F == 0) return cudaSuccess;
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3((unsigned)blocks);
    cfg.blockDim = dim3(THREADS);
    cfg.stream = st;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    cudaError_t e = diam ? cudaLaunchKernelEx(&cfg, sweep_band_kernel<K, true, THREADS, VAR>, a, g.dn_rec, g.dn_rec2,
                                              g.dn_ovf, dist, flags, diam)
                         : cudaLaunchKernelEx(&cfg, sweep_band_kernel<K, false, THREADS, VAR>, a, g.dn_rec, g.dn_rec2,
                                              g.dn_ovf, dist, flags, diam);
    count_launch();
    return e;
}

template <int K, int VAR>
cudaError_t band_kv(const DevImage& g, const BandArgs& a, const uint32_t* flags, uint32_t* dist, uint32_t* diam,
                    cudaStream_t st) {
    switch (a.threads) {
        case 128: return band_kt<K, 128, VAR>(g, a, flags, dist, diam, st);
        case 256: return band_kt<K, 256, VAR>(g, a, flags, dist, diam, st);
        default: return cudaErrorInvalidValue;
    }
}

template <int K>
cudaError_t band_k(const DevImage& g, const BandArgs& a, const uint32_t* flags, uint32_t* dist, uint32_t* diam,
                   cudaStream_t st) {
    if constexpr (K < 16) {
        return a.variant == 0 ? band_kv<K, 0>(g, a, flags, dist, diam, st) : cudaErrorInvalidValue;
    } else {
        switch (a.variant) {
            case 0: return band_kv<K, 0>(g, a, flags, dist, diam, st);
            case 1: return band_kv<K, 1>(g, a, flags, dist, diam, st);
            case 4: return band_kv<K, 4>(g, a, flags, dist, diam, st);
            case 5: return band_kv<K, 5>(g, a, flags, dist, diam, st);
            case 13: return band_kv<K, 13>(g, a, flags, dist, diam, st);
            default: return cudaErrorInvalidValue;
        }
    }
}

// ------------------------------------------------------------------ probe A33
// Sequential stream over the sweep's arrays: every ELL record read, every label row
// read and written once (no gathers, no level dependencies, ONE launch).
template <int K>
__global__ void __launch_bounds__(SWEEP_THREADS, 8)
    probe_stream_kernel(const uint4* __restrict__ rec, uint32_t* __restrict__ d, uint32_t n) {
    using T = typename RowT<K>::T;
    constexpr uint32_t G = K / RowT<K>::W;
    const uint64_t total = (uint64_t)n * G;
    for (uint64_t t = (uint64_t)blockIdx.x * SWEEP_THREADS + threadIdx.x; t < total;
         t += (uint64_t)gridDim.x * SWEEP_THREADS) {
        const uint32_t v = (uint32_t)(t / G), lane = (uint32_t)(t % G);
        const uint4 r = __ldg(&rec[v]);
        T* p = reinterpret_cast<T*>(d + (size_t)v * K) + lane;
        const T x = __ldcs(p);
        __stcs(p, relax(x, splat<T>(r.x), r.y));
    }
}

template <int K>
cudaError_t probe_stream_k(const DevImage& g, uint32_t* dist, cudaStream_t st) {
    constexpr uint32_t G = K / RowT<K>::W;
    uint64_t blocks = ((uint64_t)g.n * G + SWEEP_THREADS - 1) / SWEEP_THREADS;
    blocks = std::min<uint64_t>(blocks, (uint64_t)num_sms() * 8);
    if (blocks == 0) return cudaSuccess;
    probe_stream_kernel<K><<<(unsigned)blocks, SWEEP_THREADS, 0, st>>>(g.dn_rec, dist, g.n);
    count_launch();
    return cudaGetLastError();
}

// ------------------------------------------------------------------ a5 reductions
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

__global__ void __launch_bounds__(256) argmax_kernel(const uint32_t* __restrict__ d, uint32_t n, uint32_t k,
                                                     uint32_t kv, unsigned long long* key) {
    unsigned long long best = 0;
    const uint64_t total = (uint64_t)n * k;
    for (uint64_t t = (uint64_t)blockIdx.x * 256 + threadIdx.x; t < total; t += (uint64_t)gridDim.x * 256) {
        const uint32_t x = __ldg(&d[t]);
        if (x == INF || (uint32_t)(t % k) >= kv) continue;
        const unsigned long long c = ((unsigned long long)x << 32) | (0xFFFFFFFFu - (uint32_t)t);
        best = best > c ? best : c;
    }
    for (int o = 16; o; o >>= 1) {
        const unsigned long long y = __shfl_xor_sync(0xFFFFFFFFu, best, o);
        best = best > y ? best : y;
    }
    if ((threadIdx.x & 31) == 0 && best) atomicMax(key, best);
}

__global__ void __launch_bounds__(256) compact_kernel(const uint32_t* __restrict__ src, uint32_t ks,
                                                      uint32_t* __restrict__ dst, uint32_t kd, uint32_t n) {
    const uint64_t total = (uint64_t)n * kd;
    for (uint64_t t = (uint64_t)blockIdx.x * 256 + threadIdx.x; t < total; t += (uint64_t)gridDim.x * 256) {
        const uint64_t r = t / kd;
        __stcs(dst + t, __ldcs(src + r * ks + (t - r * kd)));
    }
}

unsigned grid_for(uint64_t items) {
    const uint64_t b = (items + 255) / 256;
    return (unsigned)std::max<uint64_t>(1, std::min<uint64_t>(b, (uint64_t)num_sms() * 8));
}

template <int K>
cudaError_t seed_k(const DevImage& g, const Slot& sl, uint32_t* dist, cudaStream_t st) {
    seed_rows_kernel<K><<<K, 256, 0, st>>>(sl, g.seed_cap, dist);
    count_launch();
    return cudaGetLastError();
}

}  // namespace

cudaError_t launch_upward(const DevImage& g, const Slot& sl, const Sources& src, uint32_t k, uint32_t vtop,
                          cudaStream_t st) {
    cudaError_t e = ensure_smem_attr((const void*)upward_kernel, (int)(5 * UP_SMEM_CAP * sizeof(uint32_t)));
    if (e != cudaSuccess) return e;
    const size_t smem = 5 * (size_t)g.smem_cap * sizeof(uint32_t);
    upward_kernel<<<k, UP_THREADS, smem, st>>>(g, sl, src, vtop);
    count_launch();
    return cudaGetLastError();
}

cudaError_t launch_seed(const DevImage& g, const Slot& sl, uint32_t k, uint32_t* dist, cudaStream_t st) {
#define CALL_SR(K) seed_k<K>(g, sl, dist, st)
    cudaError_t e = [&]() -> cudaError_t { PHAST_K_SWITCH(k, CALL_SR) }();
#undef CALL_SR
    if (e != cudaSuccess) return e;
    scatter_kernel<<<k, 256, 0, st>>>(sl, g.seed_cap, k, dist);
    count_launch();
    return cudaGetLastError();
}

cudaError_t launch_sweep_level(const DevImage& g, const uint32_t* flags, uint32_t k, uint32_t vbeg, uint32_t vend,
                               uint32_t* dist, uint32_t* diam, bool store, bool last_level, bool nogather, bool wide,
                               cudaStream_t st) {
#define CALL_SW(K) sweep_k<K>(g, flags, vbeg, vend, dist, diam, store, last_level, nogather, wide, st)
    PHAST_K_SWITCH(k, CALL_SW)
#undef CALL_SW
}

cudaError_t launch_sweep_band(const DevImage& g, const BandArgs& a, const uint32_t* flags, uint32_t k, uint32_t* dist,
                              uint32_t* diam, cudaStream_t st) {
#define CALL_BD(K) band_k<K>(g, a, flags, dist, diam, st)
    PHAST_K_SWITCH(k, CALL_BD)
#undef CALL_BD
}

uint32_t band_sm_threads(uint32_t variant, uint32_t) {
    return variant & 8 ? 1024u : variant & 1 ? 1280u : 1536u;
}

cudaError_t launch_clear_flags(const Slot& sl, uint32_t k, uint32_t seed_cap, cudaStream_t st) {
    clear_flags_kernel<<<k, 256, 0, st>>>(sl, seed_cap);
    count_launch();
    return cudaGetLastError();
}

cudaError_t launch_max_reduce(const uint32_t* in, uint32_t count, uint32_t* out, cudaStream_t st) {
    max_reduce_kernel<<<1, 1024, 0, st>>>(in, count, out);
    count_launch();
    return cudaGetLastError();
}

cudaError_t launch_argmax(const uint32_t* d, uint32_t n, uint32_t k, uint32_t kv, unsigned long long* key,
                          cudaStream_t st) {
    argmax_kernel<<<grid_for((uint64_t)n * k), 256, 0, st>>>(d, n, k, kv, key);
    count_launch();
    return cudaGetLastError();
}

cudaError_t launch_compact(const uint32_t* src, uint32_t ks, uint32_t* dst, uint32_t kd, uint32_t n,
                           cudaStream_t st) {
    compact_kernel<<<grid_for((uint64_t)n * kd), 256, 0, st>>>(src, ks, dst, kd, n);
    count_launch();
    return cudaGetLastError();
}

cudaError_t launch_probe_stream(const DevImage& g, uint32_t k, uint32_t* dist, cudaStream_t st) {
#define CALL_PR(K) probe_stream_k<K>(g, dist, st)
    PHAST_K_SWITCH(k, CALL_PR)
#undef CALL_PR
}

}  // namespace phast
