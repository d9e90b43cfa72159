// top.cu -- a3 + a4 for the top levels (or a whole small query) in ONE CTA.
//
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
#include <algorithm>

#include "device.cuh"
#include "kernels.h"

namespace phast {
namespace {

constexpr int TOP_PROD = 4;   // producer warps: one warp's cp.async stream alone starved the consumers (ncu, C1)
constexpr int TOP_THREADS = 1024, TOP_CONS = TOP_THREADS - 32 * TOP_PROD;
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
// dynamic shared memory: the 227 KB per-CTA maximum less the static heavy-vertex lists
constexpr size_t TOP_STATIC = 2 * 2 * 1024 + 64;
constexpr size_t TOP_SMEM_MAX = 227 * 1024 - TOP_STATIC;

constexpr uint32_t TOP_HEAVY = 8;              // in-arcs above which a warp relaxes the vertex (k <= 4)
constexpr uint32_t TOP_VMASK = 0x3FFFFFFFu;    // chunk vend; bit 31: the chunk has a vertex with > TOP_HEAVY
constexpr uint32_t TOP_MULTI = 0x40000000u;    // in-arcs; bit 30: a multi-level chunk (one warp, rounds)

template <int K, bool DIAM>
__global__ void __launch_bounds__(TOP_THREADS, 1) sweep_top_kernel(TopArgs A, Sources src, uint32_t* __restrict__ d,
                                                                   const uint32_t* __restrict__ flags,
                                                                   uint32_t* __restrict__ diam) {
    using T = typename RowT<K>::T;
    constexpr uint32_t G = K / RowT<K>::W;   // lanes per vertex
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
            mbar_init(&full[s], 32 * TOP_PROD);   // one cp.async arrival per producer lane
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
        for (uint32_t i = tid; i < V * G; i += TOP_THREADS) srow[i] = visited(flags, i / G) ? dr[i] : inf_row<T>();
    }
    __syncthreads();
    uint32_t mx = 0;
    if (tid < 32 * TOP_PROD) {   // producer warps: all their lanes copy (cp.async, 16 B each), then arrive
        // descriptors: each lane holds one of the current 32 and one of the next 32
        // (loaded a batch ahead), so the issue loop never waits on a global load
        const uint32_t lane = tid & 31, ptid = tid;
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
            const bool up = c < A.split;
            const uint32_t f0 = ch.x & ~3u, nf4 = ((ch.y & TOP_VMASK) + 1 - f0 + 3) / 4;   // 16-byte units
            const uint32_t a0 = ch.z & ~1u, na2 = (ch.w - a0 + 1) / 2;
            unsigned char* st = ring + (size_t)s * SB;
            const uint4* gf = reinterpret_cast<const uint4*>((up ? A.first[0] : A.first[1]) + f0);
            const uint4* ga = reinterpret_cast<const uint4*>((up ? A.arcs[0] : A.arcs[1]) + a0);
            const uint32_t nr = (ch.y & TOP_MULTI) ? 2u : 0u;   // + the rounds of a multi-level chunk
            for (uint32_t u = ptid; u < 1 + nf4 + na2 + nr; u += 32 * TOP_PROD) {
                if (u == 0) cp_async16(st, A.chunks + c);   // the consumers read the descriptor here
                else if (u <= nf4) cp_async16(st + 16 * u, gf + (u - 1));
                else if (u <= nf4 + na2) cp_async16(st + 16 + OFFB * 4 + 16 * (u - 1 - nf4), ga + (u - 1 - nf4));
                else cp_async16(st + 16 + OFFB * 4 - 32 + 16 * (u - 1 - nf4 - na2), A.rnd + 2 * c + (u - 1 - nf4 - na2));
            }
            asm volatile("cp.async.mbarrier.arrive.noinc.shared::cta.b64 [%0];" ::"r"(smem_u32(&full[s])) : "memory");
            if (++s == S) { s = 0; ph ^= 1u; }
        }
    } else {
        const uint32_t ct = tid - 32 * TOP_PROD;
        __shared__ uint32_t hcnt[2];            // heavy vertices of the chunk (double-buffered)
        __shared__ uint16_t hlist[2][TOP_VCH_BIG];   // as offsets from the chunk's first vertex
        static_assert(sizeof(hcnt) + sizeof(hlist) <= TOP_STATIC, "static shared memory");
        if (ct < 2) hcnt[ct] = 0;
        asm volatile("bar.sync 1, %0;" ::"n"(TOP_CONS) : "memory");
        uint32_t s = 0, ph = 0;
        for (uint32_t c = 0; c < A.nchunks; c++) {
            // the other count was last used by chunk c - 1, whose readers all passed its
            // end barrier; chunk c + 1's writers wait for chunk c's end barrier
            if (ct == 0) hcnt[(c + 1) & 1] = 0;
            mbar_wait(&full[s], ph);
            const unsigned char* st = ring + (size_t)s * SB;
            const uint4 ch = *reinterpret_cast<const uint4*>(st);
            const uint32_t f0 = ch.x & ~3u, a0 = ch.z & ~1u;
            const uint32_t* sf = reinterpret_cast<const uint32_t*>(st + 16);
            const uint2* sa = reinterpret_cast<const uint2*>(st + 16 + OFFB * 4);
            const uint32_t vend = ch.y & TOP_VMASK;
            const bool heavy = G == 1 && (ch.y & 0x80000000u);   // host: some vertex has > TOP_HEAVY in-arcs
            const uint32_t total = (vend - ch.x) * G;
            if (ch.y & TOP_MULTI) {
                // several tiny levels, one warp: item i (vertex ch.x + i / G) runs in round
                // rnd[i] (its level inside the chunk; every tail inside the chunk has a
                // smaller round), with only a warp barrier between rounds
                if (ct < 32) {
                    const unsigned char* rb = st + 16 + OFFB * 4 - 32;
                    const uint32_t r = ct < total ? rb[ct] : 0u;
                    const uint32_t maxr = __reduce_max_sync(0xFFFFFFFFu, r);
                    const uint32_t v = ch.x + ct / G, lane = ct % G;
                    for (uint32_t q = 0; q <= maxr; q++) {
                        if (ct < total && r == q) {
                            T acc = srow[v * G + lane];
                            for (uint32_t e = sf[v - f0], e1 = sf[v + 1 - f0]; e < e1; e++) {
                                const uint2 a = sa[e - a0];
                                acc = relax(acc, srow[a.x * G + lane], a.y);
                            }
                            srow[v * G + lane] = acc;
                        }
                        __syncwarp();
                    }
                }
            } else
            for (uint32_t t = ct; t < total; t += TOP_CONS) {
                const uint32_t v = ch.x + t / G, lane = t % G;
                const uint32_t e0 = sf[v - f0], e1 = sf[v + 1 - f0];
                if (heavy && e1 - e0 > TOP_HEAVY) {   // a warp takes it below
                    hlist[c & 1][atomicAdd(&hcnt[c & 1], 1u)] = (uint16_t)(v - ch.x);
                    continue;
                }
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
                    for (int r = 0; r < 4; r++) x[r] = e + r < e1 ? srow[a[r].x * G + lane] : inf_row<T>();   // no pad read
#pragma unroll
                    for (int r = 0; r < 4; r++) acc = relax(acc, x[r], a[r].y);
                }
                srow[v * G + lane] = acc;
            }
            if (heavy) {
                // vertices with many in-arcs (the top of G-up: every lower neighbour is
                // an in-arc) would serialise a level on one thread: one warp each, the
                // lanes striding over the arcs, then a warp min.  The light pass listed
                // them; the list is complete after this barrier (heavy chunks only).
                asm volatile("bar.sync 1, %0;" ::"n"(TOP_CONS) : "memory");
                const uint32_t wid = ct >> 5, wl = ct & 31, nh = hcnt[c & 1];
                for (uint32_t i = wid; i < nh; i += TOP_CONS / 32) {
                    const uint32_t v = ch.x + hlist[c & 1][i];
                    const uint32_t e0 = sf[v - f0], e1 = sf[v + 1 - f0];
                    T acc = wl == 0 ? srow[v] : inf_row<T>();
                    for (uint32_t e = e0 + wl; e < e1; e += 128) {   // four arcs per lane in flight
                        uint2 a[4];
                        T x[4];
#pragma unroll
                        for (int r = 0; r < 4; r++) a[r] = e + 32 * r < e1 ? sa[e + 32 * r - a0] : make_uint2(0u, INF);
#pragma unroll
                        for (int r = 0; r < 4; r++) x[r] = e + 32 * r < e1 ? srow[a[r].x] : inf_row<T>();
#pragma unroll
                        for (int r = 0; r < 4; r++) acc = relax(acc, x[r], a[r].y);
                    }
                    acc = warp_min(acc);
                    if (wl == 0) srow[v] = acc;
                }
            }
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

template <int K>
cudaError_t top_k(TopArgs A, const Sources& src, uint32_t* dist, const uint32_t* flags, uint32_t* diam,
                  cudaStream_t st) {
    const size_t lab = ((size_t)A.V * K * 4 + 15) & ~(size_t)15;
    if (lab > top_label_budget()) return cudaErrorInvalidValue;
    const size_t SB = top_stage_bytes(A.big);
    A.stages = (uint32_t)std::min<size_t>(TOP_MAX_STAGES, (TOP_SMEM_MAX - lab) / (SB + 16));
    const size_t smem = lab + A.stages * (SB + 16);
    auto kern = diam ? sweep_top_kernel<K, true> : sweep_top_kernel<K, false>;
    cudaError_t e = ensure_smem_attr((const void*)kern, (int)TOP_SMEM_MAX);
    if (e != cudaSuccess) return e;
    kern<<<1, TOP_THREADS, smem, st>>>(A, src, dist, flags, diam);
    count_launch();
    return cudaGetLastError();
}

}  // namespace

size_t top_label_budget() { return TOP_SMEM_MAX - top_ring_min() - 16; }
uint32_t top_chunk_vertices(bool big) { return big ? TOP_VCH_BIG : TOP_VCH; }
uint32_t top_chunk_arcs(bool big) { return big ? TOP_ECH_BIG : TOP_ECH; }
bool top_big_fits(uint32_t k, uint32_t V) {   // rows + 4 big stages within shared memory
    const size_t lab = ((size_t)V * k * 4 + 15) & ~(size_t)15;
    return lab + 4 * (top_stage_bytes(true) + 16) <= TOP_SMEM_MAX;
}
uint32_t top_heavy_arcs() { return TOP_HEAVY; }
uint32_t top_multi_bit() { return TOP_MULTI; }

cudaError_t launch_sweep_top(const TopArgs& A, uint32_t k, const Sources& src, uint32_t* dist,
                             const uint32_t* flags, uint32_t* diam, cudaStream_t st) {
#define CALL_TOP(K) top_k<K>(A, src, dist, flags, diam, st)
    PHAST_K_SWITCH(k, CALL_TOP)
#undef CALL_TOP
}

}  // namespace phast
