// kernels.h -- internal launch API of libphast's sm_100a kernels (not the C ABI).
//   sweep.cu : a1 upward search, a2 seeding, a3 per-level sweep, a5 reductions,
//              witness argmax, column compaction, probes A33/A34
//   top.cu   : a3 + a4 for the top levels (or a whole small query) in one CTA
//   next.cu  : NEXT-1 parent pointers, NEXT-3 betweenness / reach passes
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

namespace phast {

constexpr uint32_t INF = 0xFFFFFFFFu;
constexpr uint32_t KMAX = 64;
// per-call scratch slots: up to SLOTS queries of one handle may be in flight at once
// (each on its own stream); a call waits on the device only for the call SLOTS back
constexpr uint32_t SLOTS = 8;

// Device image of the hierarchy (static after upload; all device pointers).
struct DevImage {
    uint32_t n = 0;
    const uint32_t* dn_first = nullptr;  // [n+1]   G-down in-arcs by head (internal ids)
    const uint2* dn_arc = nullptr;       // [m_down] {tail, len}
    // G-down as ELL-2 records (the per-level sweep): rec[v] = {tail0, len0, tail1, len1};
    // len = INF marks "no arc" (arcs of length INF never exist in G-down, reading R1);
    // len1 = INF with tail1 != INF: more than two in-arcs, tail1 indexes dn_ovf = {count,
    // 0} followed by the remaining count arcs {tail, len}
    const uint4* dn_rec = nullptr;       // [n]
    // "wide" levels (capi.cu: many vertices with 3-4 in-arcs) use two records loaded
    // side by side: rec[v] = {tail0, len0, tail1, len1} and rec2[v] = {tail2, len2,
    // tail3, len3} (INF-padded); more than four in-arcs: len3 = INF with tail3 != INF
    // indexing dn_ovf = {count, 0} followed by the arcs from the fourth on
    const uint4* dn_rec2 = nullptr;      // [n] (entries of wide levels only)
    const uint2* dn_ovf = nullptr;       // [overflow entries]
    const uint32_t* up_first = nullptr;  // [n+1]   G-up out-arcs by tail
    const uint2* up_arc = nullptr;       // [m_up]   {head, len}
    uint32_t* err = nullptr;             // [1] sticky device error word (bit 0: search-space overflow)
    uint32_t seed_cap = 0;               // search-space entries per source (power of two)
    uint32_t smem_cap = 4096;            // shared-memory table entries per search (power of two, <= 4096)
};

// Per-call scratch (one per slot).
struct Slot {
    uint32_t* flags = nullptr;      // [ceil(n/32)] visited bits (§IV-C), zero between calls
    uint32_t* seed_v = nullptr;     // [KMAX][seed_cap] upward search space: vertex
    uint32_t* seed_d = nullptr;     // [KMAX][seed_cap] upward search space: label
    uint32_t* seed_cnt = nullptr;   // [KMAX]
    uint32_t* gscratch = nullptr;   // [KMAX * seed_cap * 5] global fallback tables of this slot's upward searches
};

struct Sources {
    uint32_t s[KMAX];  // internal ids, passed by value in the kernel parameter space
};

// a1: one CTA per source; exact G-up labels; the search space goes to the slot's seed
// buffers.  vtop > 0: the top levels [0, vtop) are not expanded (their labels come
// from the arcs entering them; sweep_top_kernel's G-up pull pass finishes them).
cudaError_t launch_upward(const DevImage& g, const Slot& sl, const Sources& src, uint32_t k, uint32_t vtop,
                          cudaStream_t st);
// a2: visited bits + rows of the search spaces reset to INF, then (second launch, so
// that every reset precedes every label) dist[v*k + i] = label_i(v).
cudaError_t launch_seed(const DevImage& g, const Slot& sl, uint32_t k, uint32_t* dist, cudaStream_t st);
// a3: one level [vbeg, vend) of the downward sweep; diam != nullptr fuses the max (a5);
// store == false skips the row stores (diameter mode: level-0 rows are never read);
// last_level: rows are stored evict-first (nobody reads them again).
// nogather (probe A34): every tail-row gather is replaced by the arc length itself.
// wide: the level's records are in the two-record format (DevImage::dn_rec2).
cudaError_t launch_sweep_level(const DevImage& g, const uint32_t* flags, uint32_t k, uint32_t vbeg, uint32_t vend,
                               uint32_t* dist, uint32_t* diam, bool store, bool last_level, bool nogather, bool wide,
                               cudaStream_t st);
// a3 for a band of levels (layout.h Band) in ONE launch: work unit u (consecutive
// closed groups) of level j (j = 0 the band's top level) is the id range [off[j*(U+1)
// + u], off[j*(U+1) + u + 1]); one CTA sweeps a unit level by level (a CTA barrier
// between levels, none between units: groups share no in-band arcs).  Rows of the
// unit's upper levels are read back by its lower levels from L2.
struct BandArgs {
    const uint32_t* off = nullptr;   // device [F][U+1]
    uint32_t F = 0, U = 0;
    uint32_t wide = 0;               // bit j: level j uses the two-record format (DevImage::dn_rec2)
    uint32_t store_last = 1;         // 0: the band's last level is not stored (diameter mode, CH level 0)
    uint32_t stream_last = 0;        // 1: the last level's rows are stored evict-first (never read again)
    uint32_t threads = 128;          // CTA size: 128 or 256
    uint32_t variant = 0;            // sweep.cu band kernel variants (bits: PF_REG, PF_L2, FULL)
};
cudaError_t launch_sweep_band(const DevImage& g, const BandArgs& a, const uint32_t* flags, uint32_t k, uint32_t* dist,
                              uint32_t* diam, cudaStream_t st);
// resident threads of the band kernel per SM (its grid is at most num_sms() * this / threads)
uint32_t band_sm_threads(uint32_t variant, uint32_t threads);
// after the sweep: clear the visited bits of every search-space vertex ("After
// scanning v we unmark the vertex", §IV-C).
cudaError_t launch_clear_flags(const Slot& sl, uint32_t k, uint32_t seed_cap, cudaStream_t st);

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
    // multi-level chunks (vend bit 30, top_multi_bit()): several tiny consecutive levels
    // whose (vertex, lane) items fit one warp; rnd[2c..2c+1] = 32 bytes, byte i = the
    // round (level inside the chunk, 0 first) of the chunk's i-th item's vertex
    const uint4* rnd = nullptr;
};
cudaError_t launch_sweep_top(const TopArgs& A, uint32_t k, const Sources& src, uint32_t* dist,
                             const uint32_t* flags, uint32_t* diam, cudaStream_t st);
size_t top_label_budget();
uint32_t top_chunk_vertices(bool big);
uint32_t top_chunk_arcs(bool big);
bool top_big_fits(uint32_t k, uint32_t V);   // the big geometry leaves room for the rows
uint32_t top_heavy_arcs();   // chunk flag (bit 31 of vend): some vertex has more in-arcs than this
uint32_t top_multi_bit();    // chunk flag (bit 30 of vend): a multi-level chunk (TopArgs::rnd)

// a5: max of `count` per-batch maxima into *out
cudaError_t launch_max_reduce(const uint32_t* in, uint32_t count, uint32_t* out, cudaStream_t st);
// diameter witness: *key = max over items t = r*k + i (i < kv) with d[t] != INF of
// (d[t] << 32 | (2^32-1 - t)): the largest finite label, ties to the smallest item.
// *key must be zeroed before (n*k < 2^32).
cudaError_t launch_argmax(const uint32_t* d, uint32_t n, uint32_t k, uint32_t kv, unsigned long long* key,
                          cudaStream_t st);
// dst[r*kd + i] = src[r*ks + i] for i < kd (a query computed at a padded width ks)
cudaError_t launch_compact(const uint32_t* src, uint32_t ks, uint32_t* dst, uint32_t kd, uint32_t n,
                           cudaStream_t st);
// probe A33 (§VIII-B "this takes 65.6 ms; PHAST is only 2.6 times slower
// than this"): read every ELL record and every label row and write every row once, in
// sequential order -- the bytes of the sweep without its gathers and dependencies.
cudaError_t launch_probe_stream(const DevImage& g, uint32_t k, uint32_t* dist, cudaStream_t st);

// NEXT-1 parent pointers (§VII-A "we check whether the identity d(v) =
// d(u) + l(u,v) holds"): parent[r*k + i] = internal id of the tail of the first
// (smallest input index) original arc (u, v) with d_i(u) + l = d_i(v); the source's
// own row entry is itself; INF where d_i(v) = INF.  in_first/in_arc: the original
// graph's in-CSR in internal ids (Layout::in_first / in_arc).  Any 1 <= k <= 64.
cudaError_t launch_parents(const uint32_t* in_first, const uint2* in_arc, uint32_t n, const Sources& src,
                           uint32_t k, const uint32_t* dist, uint32_t* parent, cudaStream_t st);

// NEXT-1 parent pointers in the hierarchy G+ = A-down U A-up (reading R19): parent[r*k +
// i] = the tail of v's first tight A-down in-arc (dn_first/dn_arc order), else of its
// first tight A-up in-arc (upin: A-up in-arcs by head, tails increasing); the source's
// own entry is itself; INF where d_i(v) = INF.  Any 1 <= k <= 64.
cudaError_t launch_parents_ch(const uint32_t* dn_first, const uint2* dn_arc, const uint32_t* upin_first,
                              const uint2* upin_arc, uint32_t n, const Sources& src, uint32_t k, const uint32_t* dist,
                              uint32_t* parent, cudaStream_t st);

// NEXT-3 betweenness / reach (next.cu): passes in Kahn order of each tree's tight DAG;
// items t = v*k + i (n*k < 2^32).
struct BcGraph {
    const uint32_t* in_first;   // original in-arcs by head {tail, len}, internal ids
    const uint2* in_arc;
    const uint32_t* out_first;  // original out-arcs by tail {head, len}
    const uint2* out_arc;
    uint32_t* err;              // sticky device error word: bit 0 if a path count exceeds 2^53
};
struct BcQueue {
    const uint32_t* q_in;       // items of this pass
    const uint32_t* qs_in;      // their count
    uint32_t* q_out;            // items that become ready
    uint32_t* qs_out;
    uint32_t* qs_clr;           // counter zeroed for the pass after next
    uint32_t* cnt;              // [n*k] unfinished inputs per item
};
// B batches of k trees at once: arrays [B][n][k], nk = n*k, total = B*nk items (< 2^32).
// Forward count (backward = 0) computes the tight-arc masks min_/mout of every item and
// the forward counts; the backward count only popcounts mout (call it after).
cudaError_t launch_bc_count(const BcGraph& G, const uint32_t* d, uint32_t nk, uint32_t k, uint32_t total, int backward,
                            uint32_t* cnt, uint32_t* min_, uint32_t* mout, uint32_t* q, uint32_t* qs, cudaStream_t st);
cudaError_t launch_bc_sigma(const BcGraph& G, const uint32_t* d, double* sigma, uint32_t nk, uint32_t k,
                            uint32_t total, const uint32_t* min_, const uint32_t* mout, const BcQueue& Q,
                            uint32_t* changed, cudaStream_t st);
cudaError_t launch_bc_back(const BcGraph& G, const uint32_t* d, const double* sigma, void* val, uint32_t nk,
                           uint32_t k, uint32_t total, const uint32_t* min_, const uint32_t* mout, int mode,
                           const BcQueue& Q, uint32_t* changed, cudaStream_t st);
// accumulation over trees j = b*k + i < valid; src: DEVICE internal ids of the trees
cudaError_t launch_reach_accum(const uint32_t* d, const uint32_t* hgt, uint32_t* r, uint32_t n, uint32_t k,
                               uint32_t valid, cudaStream_t st);
cudaError_t launch_bc_accum(const double* delta, double* cb, uint32_t n, uint32_t k, uint32_t valid,
                            const uint32_t* src, cudaStream_t st);

uint64_t launches();
// kernels replayed from a CUDA graph (counted at launch, not at capture)
void add_launches(int64_t d);
void count_launch();
// SM count of the current device (cached per device ordinal)
int num_sms();
// cudaFuncSetAttribute(MaxDynamicSharedMemorySize) once per (kernel, device)
cudaError_t ensure_smem_attr(const void* kernel, int bytes);

}  // namespace phast
