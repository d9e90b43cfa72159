// kernels.h -- internal launch API of libphast's sm_100a kernels (not the C ABI).
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

namespace phast {

constexpr uint32_t INF = 0xFFFFFFFFu;
constexpr uint32_t KMAX = 64;
constexpr uint32_t SEED_SLOTS = 2;

// Device image of the hierarchy + per-handle scratch (all device pointers).
struct DevImage {
    uint32_t n = 0;
    const uint32_t* dn_first = nullptr;  // [n+1]   G-down in-arcs by head (internal ids)
    const uint2* dn_arc = nullptr;       // [m_down] {tail, len}
    // G-down as ELL-2 records (the per-level sweep's default): rec[v] = {tail0, len0,
    // tail1, len1}; len = INF marks "no arc" (arcs of length INF never exist in G-down,
    // reading R1); len1 = INF with tail1 != INF: more than two in-arcs, tail1 indexes
    // dn_ovf = {count, 0} followed by the remaining count arcs {tail, len}
    const uint4* dn_rec = nullptr;       // [n]
    const uint2* dn_ovf = nullptr;       // [overflow entries]
    const uint32_t* up_first = nullptr;  // [n+1]   G-up out-arcs by tail
    const uint2* up_arc = nullptr;       // [m_up]   {head, len}
    uint32_t* flags = nullptr;           // [ceil(n/32)] visited bits (§IV-C), zero between calls
    const uint32_t* tail_bits = nullptr; // [ceil(n/32)] bit v: v is the tail of some G-down arc
    uint32_t* seed_v = nullptr;          // [SEED_SLOTS][KMAX][seed_cap] upward search spaces: vertex
    uint32_t* seed_d = nullptr;          // [SEED_SLOTS][KMAX][seed_cap] upward search spaces: label
    uint32_t* seed_cnt = nullptr;        // [SEED_SLOTS][KMAX]
    uint32_t* gscratch = nullptr;        // [KMAX * seed_cap * 5] global-memory fallback tables
    uint32_t* err = nullptr;             // [1] sticky device error word
    uint32_t seed_cap = 0;               // entries per source (power of two)
    uint32_t smem_cap = 4096;            // shared-memory table entries (power of two, <= 4096)
};

struct Sources {
    uint32_t s[KMAX];  // internal ids, passed by value in the kernel parameter space
};

// a1: one CTA per source; exact G-up labels; the search space goes to seed slot `slot`
// (SEED_SLOTS slots, so the next batch's searches can run beside this batch's sweep).
// vtop > 0: the top levels [0, vtop) are not expanded (their labels come from the
// arcs entering them; sweep_top_kernel's G-up pull pass finishes them).
cudaError_t launch_upward(const DevImage& g, const Sources& src, uint32_t k, uint32_t slot, uint32_t vtop,
                          cudaStream_t st);
// a2: visited bits + rows of the search spaces reset to INF, then (second launch, so
// that every reset precedes every label) dist[v*k + i] = label_i(v).
cudaError_t launch_seed(const DevImage& g, uint32_t k, uint32_t slot, uint32_t* dist, cudaStream_t st);
// a3: one level [vbeg, vend) of the downward sweep; diam != nullptr fuses the max (a5);
// store == false skips the row stores (diameter mode, level 0 rows are never read).
// by_tail: the segment mixes levels; store each row by its tail bit (tails normally,
// others evict-first; diameter: others not stored).
cudaError_t launch_sweep_level(const DevImage& g, uint32_t k, uint32_t vbeg, uint32_t vend,
                               uint32_t* dist, uint32_t* diam, bool store, bool last_level,
                               bool by_tail, cudaStream_t st);
// Plan of the persistent (single-launch) sweep for one k: the internal order is cut
// into chunks of consecutive ids (no chunk contains both ends of a G-down arc);
// chunk c runs on CTA c % grid in iteration c / grid and depends on iteration
// chunk_dep[c] - 1 (0 = no dependency).
struct SweepPlan {
    uint32_t k = 0, nchunks = 0, grid = 0, iters = 0, chunk_cap = 0;
    uint32_t variant = 2;   // 6: segment barriers (chunk_v = segment offsets, nchunks = segments,
                            //    chunk_cap = first segment stored by tail bit, wave_done = per-segment counters);
                            // 5: warp waves (wave plan, per-wave sub-counters); 4: warp pipeline; 3: pipelined gather; 2: warp dataflow; 1: CTA waves + bulk-staged arcs; 0: CTA waves
    // variant 3 (pipelined gather): per slot {vbeg, vend, e0 = first[vbeg], e1 = first[vend]}
    const uint4* pinfo = nullptr;
    // variant 2 (warp dataflow)
    uint32_t workers = 0;                   // warps in the grid
    const uint4* wmeta = nullptr;           // [nchunks] {vbeg, vend, dbeg, dend}
    const uint32_t* wdeps = nullptr;        // dependency chunk ids
    uint32_t* done = nullptr;               // [nchunks] epoch of the last completion
    const uint32_t* chunk_v = nullptr;      // [nchunks+1] chunk boundaries
    const uint32_t* chunk_dep = nullptr;    // [nchunks]
    uint32_t* wave_done = nullptr;          // [iters] monotone completion counters (epochs);
                                            // variant 5: [8][chunk_cap] sub-counters, chunk_cap = stride
    const uint4* wdesc = nullptr;           // variant 5: [iters * workers] chunk descriptors (plan_waves)
    uint32_t* err = nullptr;                // sticky device error word (bit 1: dependency watchdog)
    uint32_t stream_last = 1;               // variant 6: the last segment's rows are nobody's tail
    uint32_t seg_lag = 1;                   // variant 6: segment j waits for segment j - seg_lag (1: barrier)
};
// vertices per chunk and CTAs per SM the persistent sweep uses for this k
uint32_t sweep_chunk_vertices(uint32_t k);   // max vertices per chunk
uint32_t sweep_pass_vertices(uint32_t k);    // vertices per pass of a CTA
uint32_t sweep_warp_chunk_vertices(uint32_t k);
uint32_t sweep_wpipe_chunk_vertices(uint32_t k);  // variant 4
uint32_t sweep_wave_chunk_vertices(uint32_t k);   // variant 5: vertices per chunk
uint32_t sweep_wave_chunk_arcs();                 // variant 5: max G-down arcs per chunk (staged)
uint32_t sweep_wave_subcounters();                // variant 5: completion sub-counters per wave
constexpr uint32_t SWEEP_WARPS = 8;               // warps per CTA of the persistent sweeps
// variant 3: max vertices and arcs per chunk for k (k >= 4; 0 otherwise)
void sweep_pipe_geometry(uint32_t k, uint32_t* cap_vertices, uint32_t* cap_arcs);   // vertices per chunk of one warp (variant 2)
int sweep_blocks_per_sm(uint32_t k, bool diam, uint32_t variant);
// a3 + a4 in ONE launch: dataflow over levels through the completion counters
// (epoch = number of launches of this plan so far, 1-based).
cudaError_t launch_sweep_persistent(const DevImage& g, const SweepPlan& p, uint32_t epoch, uint32_t* dist,
                                    uint32_t* diam, cudaStream_t st);

// NEXT-1 parent pointers (§VII-A "we check whether the identity d(v) =
// d(u) + l(u,v) holds"): parent[r*k + i] = internal id of the tail of the first
// (smallest input index) original arc (u, v) with d_i(u) + l = d_i(v); the source's
// own row entry is itself; INF where d_i(v) = INF.  in_first/in_arc: the original
// graph's in-CSR in internal ids (Layout::in_first / in_arc).
cudaError_t launch_parents(const uint32_t* in_first, const uint2* in_arc, uint32_t n, const Sources& src,
                           uint32_t k, const uint32_t* dist, uint32_t* parent, cudaStream_t st);

// a3 + a4 for the top levels [0, V) in ONE single-CTA launch (labels in shared
// memory, arcs streamed by cp.async through an mbarrier ring).  chunks[c] = {vbeg, vend,
// first[vbeg], first[vend]} over CSR first[0]/arcs[0] for c < split (fused mode: the
// G-up pull sweep, ascending levels) and CSR first[1]/arcs[1] after (G-down,
// descending levels); at most top_chunk_vertices() vertices and top_chunk_arcs() arcs
// each, never spanning two levels; V * k * 4 <= top_label_budget().
//   fused = 0: rows start from the seeded rows / visited bits (after a1, a2);
//   fused = 1: V = n, rows start at INF with d_i(src.s[i]) = 0 -- the whole query
//   (a1 as a pull sweep of G-up, a2, a3) in one launch.
struct TopArgs {
    const uint32_t* first[2] = {nullptr, nullptr};
    const uint2* arcs[2] = {nullptr, nullptr};
    const uint4* chunks = nullptr;
    uint32_t split = 0, nchunks = 0, V = 0, stages = 0, fused = 0;
    uint32_t big = 0;                    // chunk geometry: 0 = top_chunk_*(false), 1 = top_chunk_*(true)
    unsigned long long* dbg = nullptr;   // diagnostics (PHAST_TOP_DEBUG): per chunk 4 clock64 stamps: consumer wait start, data ready, work done; producer issue
};
cudaError_t launch_sweep_top(const TopArgs& A, uint32_t k, const Sources& src, uint32_t* dist,
                             const uint32_t* flags, uint32_t* diam, cudaStream_t st);
size_t top_label_budget();
uint32_t top_chunk_vertices(bool big);
uint32_t top_chunk_arcs(bool big);
bool top_big_fits(uint32_t k, uint32_t V);   // the big geometry leaves room for the rows
uint32_t top_heavy_arcs();   // chunk flag (bit 31 of vend): some vertex has more in-arcs than this

// a3 + a4 for the mid levels seg[0..nseg] (device array of nseg+1 internal-id offsets,
// level-ordered) in ONE thread-block-cluster launch with a cluster barrier per level
// (ELL-2 records; needs dn_rec).  cluster_threads(): threads of the launch, 0 = disabled.
cudaError_t launch_sweep_cluster(const DevImage& g, uint32_t k, const uint32_t* seg, uint32_t nseg, uint32_t* dist,
                                 uint32_t* diam, cudaStream_t st);
uint32_t cluster_threads();

// after the sweep: clear the visited bits of every search-space vertex ("After
// scanning v we unmark the vertex", §IV-C).
cudaError_t launch_clear_flags(const DevImage& g, uint32_t k, uint32_t slot, cudaStream_t st);
// max of per-batch maxima (diameter)
cudaError_t launch_max_reduce(const uint32_t* in, uint32_t count, uint32_t* out, cudaStream_t st);

// NEXT-3 betweenness (kernels.cu): one in-place relaxation pass each; *changed := 1 if
// the pass wrote anything.  accum: cb[v] += sum_{i < kv, src.s[i] != v} delta[v*k+i].
// Passes in Kahn order of each tree's tight DAG (kernels.cu): items t = v*k + i (n*k < 2^32).
struct BcGraph {
    const uint32_t* in_first;   // original in-arcs by head {tail, len}, internal ids
    const uint2* in_arc;
    const uint32_t* out_first;  // original out-arcs by tail {head, len}
    const uint2* out_arc;
};
struct BcQueue {
    const uint32_t* q_in;       // items of this pass
    const uint32_t* qs_in;      // their count
    uint32_t* q_out;            // items that become ready
    uint32_t* qs_out;
    uint32_t* qs_clr;           // counter zeroed for the pass after next
    uint32_t* cnt;              // [n*k] unfinished inputs per item
};
cudaError_t launch_bc_count(const BcGraph& G, const uint32_t* d, uint32_t n, uint32_t k, int backward, uint32_t* cnt,
                            uint32_t* q, uint32_t* qs, cudaStream_t st);
cudaError_t launch_bc_sigma(const BcGraph& G, const uint32_t* d, double* sigma, uint32_t n, uint32_t k,
                            const BcQueue& Q, uint32_t* changed, cudaStream_t st);
cudaError_t launch_bc_back(const BcGraph& G, const uint32_t* d, const double* sigma, void* val, uint32_t n, uint32_t k,
                           int mode, const BcQueue& Q, uint32_t* changed, cudaStream_t st);
// all passes of one direction in one cooperative launch (mode 0 sigma, 1 delta, 2 height);
// queue 0 / qs[0] hold the count kernel's items; err bit 1 if max_passes is exceeded
cudaError_t launch_bc_persistent(const BcGraph& G, const uint32_t* d, double* sigma, void* val, uint32_t k, int mode,
                                 uint32_t* q0, uint32_t* q1, uint32_t* qs, uint32_t* cnt, uint32_t max_passes,
                                 uint32_t* err, cudaStream_t st);
cudaError_t launch_reach_accum(const uint32_t* d, const uint32_t* hgt, uint32_t* r, uint32_t n, uint32_t k, uint32_t kv,
                               cudaStream_t st);
cudaError_t launch_bc_accum(const double* delta, double* cb, uint32_t n, uint32_t k, uint32_t kv, const Sources& src,
                            cudaStream_t st);

uint64_t launches();
// kernels replayed from a CUDA graph (counted at launch, not at capture)
void add_launches(int64_t d);
int num_sms();
// L2 persistence for the sweep launches: the first `bytes` of each label array (the
// top levels' rows) are accessed with the persisting property; sets the device's
// persisting-L2 limit (process-wide).  0 = off.  Returns 0, or -1 if unsupported.
int set_l2_persist(size_t bytes);

}  // namespace phast
