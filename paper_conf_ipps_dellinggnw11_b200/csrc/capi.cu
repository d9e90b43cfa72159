// capi.cu -- the C ABI of include/phast.h: handle lifetime, validation, device
// image upload, sweep plans and query orchestration.
//
// Layout (layout.cpp): internal ids follow a reverse topological order
// of G-down, so that the sweep is "a simple linear sweep in increasing order of IDs"
// (§IV-A).  G-down: in-arcs by head, {tail, len} (§IV-A),
// sentinel dn_first[n].  G-up: out-arcs by tail, {head, len}.
#include <algorithm>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <map>
#include <memory>
#include <new>
#include <vector>

#include "../../include/phast.h"
#include "ch.h"
#include "kernels.h"
#include "layout.h"

using namespace phast;

struct phast_ctx {
    uint32_t n = 0;
    uint64_t m = 0, shortcuts = 0;
    uint32_t rounds = 0;
    double build_seconds = 0;
    Layout L;
    std::vector<uint32_t> tail_bits;   // bit v: internal id v is the tail of some G-down arc
    // device
    int device = -1;
    DevImage g;
    uint32_t* dist_scratch = nullptr;   // phast_trees_host / phast_diameter label buffer
    size_t dist_scratch_elems = 0;
    uint32_t* batch_max_scratch = nullptr;
    size_t batch_max_elems = 0;
    uint32_t* d_in_first = nullptr;     // original in-CSR on the device (parents; uploaded on first use)
    uint2* d_in_arc = nullptr;
    // NEXT-3 betweenness: original out-CSR {head, len} by tail (internal ids), sigma/delta
    // rows [n][k] fp64, per-pass change words (device + pinned host)
    uint32_t* d_out_first = nullptr;
    uint2* d_out_arc = nullptr;
    double* bc_sigma = nullptr;
    double* bc_delta = nullptr;
    size_t bc_elems = 0;
    uint32_t* bc_changed = nullptr;
    uint32_t* bc_changed_host = nullptr;
    uint32_t* bc_q = nullptr;           // [3][n*k]: two item queues + unfinished-input counts
    uint32_t* bc_qs = nullptr;          // [3] rotating queue sizes
    cudaStream_t bc_stream = nullptr;   // private stream the pass graphs run on
    cudaEvent_t bc_ev = nullptr;
    int bc_len_ok = 0;                  // 0 unknown, 1 all original lengths > 0, -1 not
    // persistent-sweep plans, one per k (built on first use)
    struct Plan {
        SweepPlan p;
        uint32_t epoch = 0;
        uint32_t top_levels = 0;   // hybrid (per-level mode): levels [0, top_levels) run as one persistent launch
        uint32_t bottom_from = 0;  // diagonal layout: segments [bottom_from, end) run as one lagged persistent launch
        bool ok = false;
    };
    std::map<uint32_t, Plan> plans;
    // top levels [0, J) swept in one single-CTA launch (launch_sweep_top), one plan per k
    struct Top {
        uint4* chunks = nullptr;   // device [nchunks] {vbeg, vend, first[vbeg], first[vend]}
        TopArgs a;                 // a.fused: the whole query in this one launch
        uint32_t J = 0;            // segments [0, J) in the shared-memory launch (0: none)
        uint32_t J2 = 0;           // segments [J, J2) in one cluster launch (launch_sweep_cluster)
        uint32_t* cl_seg = nullptr;   // device [J2 - J + 1] offsets
        uint32_t vtop = 0;            // upward searches stop expanding below this id (0: full searches)
        uint32_t* up_f = nullptr;     // top mode with vtop: A-up in-arcs by head inside [0, V)
        uint2* up_a = nullptr;
        bool ok = false;
    };
    std::map<uint32_t, Top> tops;
    // A-up in-arcs by head {tail, len} (fused single-launch queries on small graphs)
    uint32_t* d_upin_first = nullptr;
    uint2* d_upin_arc = nullptr;
    bool upin_tried = false;
    // 0 = warp pipeline (default), 1 = one launch per level, 2 = CTA waves, 3 = CTA waves + bulk-staged
    // arcs, 4 = pipelined CTA gather (k >= 4; else warp pipeline), 5 = warp dataflow without pipeline
    int sweep_mode = 0;
    // upward searches run on a side stream, one seed slot ahead of the sweep
    cudaStream_t side = nullptr;
    cudaEvent_t up_done[SEED_SLOTS] = {};
    cudaEvent_t slot_free[SEED_SLOTS] = {};
    uint32_t slot_next = 0;
    // stage timing (phast_timing)
    bool timing = false;
    std::vector<cudaEvent_t> ev;   // 3 per recorded batch
    size_t ev_used = 0;
};

namespace {

constexpr uint32_t SEED_CAP = 1u << 16;   // per-source search-space capacity (global fallback)
constexpr uint32_t DEFAULT_DELTA = 65536;

bool k_ok(uint32_t k) { return k == 1 || k == 2 || k == 4 || k == 8 || k == 16 || k == 32 || k == 64; }

struct DeviceGuard {
    int prev = -1;
    bool ok = true;
    explicit DeviceGuard(int dev) {
        if (cudaGetDevice(&prev) != cudaSuccess) { ok = false; return; }
        if (prev != dev && cudaSetDevice(dev) != cudaSuccess) ok = false;
    }
    ~DeviceGuard() {
        int cur = -1;
        if (prev >= 0 && cudaGetDevice(&cur) == cudaSuccess && cur != prev) cudaSetDevice(prev);
    }
};

template <class T>
int dmalloc(T** p, size_t elems) {
    *p = nullptr;
    if (elems == 0) elems = 1;
    cudaError_t e = cudaMalloc((void**)p, elems * sizeof(T));
    if (e != cudaSuccess) {
        cudaGetLastError();
        *p = nullptr;
        return e == cudaErrorMemoryAllocation ? PHAST_ENOMEM : PHAST_ECUDA;
    }
    return PHAST_OK;
}

void free_plans(phast_ctx* h) {
    for (auto& kv : h->plans) {
        cudaFree((void*)kv.second.p.chunk_v);
        cudaFree((void*)kv.second.p.chunk_dep);
        cudaFree(kv.second.p.wave_done);
        cudaFree((void*)kv.second.p.wmeta);
        cudaFree((void*)kv.second.p.pinfo);
        cudaFree((void*)kv.second.p.wdeps);
        cudaFree(kv.second.p.done);
    }
    h->plans.clear();
    for (auto& kv : h->tops) {
        cudaFree(kv.second.chunks); cudaFree(kv.second.cl_seg);
        cudaFree(kv.second.up_f); cudaFree(kv.second.up_a);
    }
    h->tops.clear();
}

void free_device(phast_ctx* h) {
    if (h->device < 0) return;
    DeviceGuard dg(h->device);
    cudaDeviceSynchronize();
    free_plans(h);
    for (cudaEvent_t e : h->ev) cudaEventDestroy(e);
    h->ev.clear();
    h->ev_used = 0;
    for (uint32_t s = 0; s < SEED_SLOTS; s++) {
        if (h->up_done[s]) cudaEventDestroy(h->up_done[s]);
        if (h->slot_free[s]) cudaEventDestroy(h->slot_free[s]);
        h->up_done[s] = h->slot_free[s] = nullptr;
    }
    if (h->side) cudaStreamDestroy(h->side);
    h->side = nullptr;
    cudaFree((void*)h->g.dn_first); cudaFree((void*)h->g.dn_arc);
    cudaFree((void*)h->g.dn_rec); cudaFree((void*)h->g.dn_ovf);
    cudaFree((void*)h->g.up_first); cudaFree((void*)h->g.up_arc);
    cudaFree(h->g.flags); cudaFree((void*)h->g.tail_bits);
    cudaFree(h->g.seed_v); cudaFree(h->g.seed_d); cudaFree(h->g.seed_cnt);
    cudaFree(h->g.gscratch); cudaFree(h->g.err);
    cudaFree(h->dist_scratch); cudaFree(h->batch_max_scratch);
    cudaFree(h->d_in_first); cudaFree(h->d_in_arc);
    h->d_in_first = nullptr; h->d_in_arc = nullptr;
    cudaFree(h->d_out_first); cudaFree(h->d_out_arc); cudaFree(h->bc_sigma); cudaFree(h->bc_delta);
    cudaFree(h->bc_changed); cudaFreeHost(h->bc_changed_host); cudaFree(h->bc_q); cudaFree(h->bc_qs);
    h->bc_q = nullptr; h->bc_qs = nullptr;
    if (h->bc_stream) cudaStreamDestroy(h->bc_stream);
    if (h->bc_ev) cudaEventDestroy(h->bc_ev);
    h->bc_stream = nullptr; h->bc_ev = nullptr;
    h->d_out_first = nullptr; h->d_out_arc = nullptr; h->bc_sigma = h->bc_delta = nullptr;
    h->bc_elems = 0; h->bc_changed = nullptr; h->bc_changed_host = nullptr;
    cudaFree(h->d_upin_first); cudaFree(h->d_upin_arc);
    h->d_upin_first = nullptr; h->d_upin_arc = nullptr;
    h->upin_tried = false;
    h->g = DevImage();
    h->dist_scratch = nullptr; h->batch_max_scratch = nullptr;
    h->dist_scratch_elems = 0; h->batch_max_elems = 0;
    h->device = -1;
}

void compute_tail_bits(phast_ctx* h) {
    h->tail_bits.assign(((size_t)h->n + 31) / 32, 0u);
    for (const Arc& a : h->L.dn_arc) h->tail_bits[a.x >> 5] |= 1u << (a.x & 31);
}

int upload(phast_ctx* h) {
    int dev = 0;
    if (cudaGetDevice(&dev) != cudaSuccess) { cudaGetLastError(); return PHAST_ECUDA; }
    h->device = dev;
    DevImage& g = h->g;
    g.n = h->n;
    if (const char* e = std::getenv("PHAST_SWEEP"))
        h->sweep_mode = std::strcmp(e, "levels") == 0       ? 1
                        : std::strcmp(e, "persistent") == 0 ? 2
                        : std::strcmp(e, "staged") == 0     ? 3
                        : std::strcmp(e, "pipe") == 0       ? 4
                        : std::strcmp(e, "warp") == 0       ? 5
                        : std::strcmp(e, "wave") == 0       ? 6
                        : std::strcmp(e, "segments") == 0   ? 7
                                                            : 0;
    // level layouts default to one launch per level (the fastest schedule measured on them)
    if (!std::getenv("PHAST_SWEEP") && !h->L.lvl_off.empty()) h->sweep_mode = 1;
    if ((h->sweep_mode == 1 || h->sweep_mode == 7) && h->L.lvl_off.empty()) h->sweep_mode = 0;   // needs segments
    // test knobs (rounded down to powers of two): shrink the shared-memory table / the
    // per-source capacity to exercise the global fallback and the overflow error path
    uint32_t seed_cap = SEED_CAP, smem_cap = 4096;
    if (const char* e = std::getenv("PHAST_SEED_CAP"))
        seed_cap = std::max(16u, std::min<uint32_t>(SEED_CAP, (uint32_t)std::atoi(e)));
    if (const char* e = std::getenv("PHAST_L2_PERSIST_MB"))   // experiment knob
        set_l2_persist((size_t)std::max(0, std::atoi(e)) << 20);
    if (const char* e = std::getenv("PHAST_UP_SMEM_CAP"))
        smem_cap = std::max(16u, std::min<uint32_t>(4096u, (uint32_t)std::atoi(e)));
    auto pow2 = [](uint32_t x) { uint32_t p = 1; while (p * 2 <= x) p *= 2; return p; };
    g.seed_cap = pow2(seed_cap);
    g.smem_cap = pow2(smem_cap);
    const Layout& L = h->L;
    uint32_t *dnf = nullptr, *upf = nullptr, *tb = nullptr;
    uint2 *dna = nullptr, *upa = nullptr;
    int rc;
    size_t nw = ((size_t)h->n + 31) / 32;
    // +4 / +2 elements: 16-byte aligned bulk copies may read up to 12 bytes past the end
    if ((rc = dmalloc(&dnf, L.dn_first.size() + 4)) || (rc = dmalloc(&dna, L.dn_arc.size() + 2)) ||
        (rc = dmalloc(&upf, L.up_first.size())) || (rc = dmalloc(&upa, L.up_arc.size())) ||
        (rc = dmalloc(&g.flags, nw)) || (rc = dmalloc(&tb, nw)) ||
        (rc = dmalloc(&g.seed_v, (size_t)SEED_SLOTS * KMAX * g.seed_cap)) ||
        (rc = dmalloc(&g.seed_d, (size_t)SEED_SLOTS * KMAX * g.seed_cap)) ||
        (rc = dmalloc(&g.seed_cnt, SEED_SLOTS * KMAX)) || (rc = dmalloc(&g.gscratch, (size_t)KMAX * g.seed_cap * 5)) ||
        (rc = dmalloc(&g.err, 1))) {
        g.dn_first = dnf; g.dn_arc = dna; g.up_first = upf; g.up_arc = upa; g.tail_bits = tb;
        free_device(h);
        return rc;
    }
    g.dn_first = dnf; g.dn_arc = dna; g.up_first = upf; g.up_arc = upa; g.tail_bits = tb;
    // G-down as ELL-2 records + overflow lists (kernels.h: DevImage::dn_rec)
    {
        std::vector<uint4> rec(h->n);
        std::vector<Arc> ovf;
        for (uint32_t v = 0; v < h->n; v++) {
            const uint32_t e0 = L.dn_first[v], deg = L.dn_first[v + 1] - e0;
            uint4 r = make_uint4(INF, INF, INF, INF);
            if (deg >= 1) { r.x = L.dn_arc[e0].x; r.y = L.dn_arc[e0].y; }
            if (deg == 2) { r.z = L.dn_arc[e0 + 1].x; r.w = L.dn_arc[e0 + 1].y; }
            if (deg > 2) {
                r.z = (uint32_t)ovf.size();
                ovf.push_back(Arc{deg - 1, 0});
                for (uint32_t e = e0 + 1; e < e0 + deg; e++) ovf.push_back(L.dn_arc[e]);
            }
            rec[v] = r;
        }
        uint4* dr = nullptr;
        uint2* dov = nullptr;
        if (ovf.size() >= INF || (rc = dmalloc(&dr, rec.size())) || (rc = dmalloc(&dov, ovf.size()))) {
            cudaFree(dr);
            free_device(h);
            return rc ? rc : PHAST_ERANGE;
        }
        g.dn_rec = dr;
        g.dn_ovf = dov;
        if (cudaMemcpy(dr, rec.data(), rec.size() * sizeof(uint4), cudaMemcpyHostToDevice) != cudaSuccess ||
            (!ovf.empty() && cudaMemcpy(dov, ovf.data(), ovf.size() * 8, cudaMemcpyHostToDevice) != cudaSuccess)) {
            cudaGetLastError();
            free_device(h);
            return PHAST_ECUDA;
        }
    }
    bool ok = cudaMemset(dnf, 0, (L.dn_first.size() + 4) * 4) == cudaSuccess &&
              cudaMemset(dna, 0, (L.dn_arc.size() + 2) * 8) == cudaSuccess &&
              cudaMemcpy(dnf, L.dn_first.data(), L.dn_first.size() * 4, cudaMemcpyHostToDevice) == cudaSuccess &&
              cudaMemcpy(dna, L.dn_arc.data(), L.dn_arc.size() * 8, cudaMemcpyHostToDevice) == cudaSuccess &&
              cudaMemcpy(upf, L.up_first.data(), L.up_first.size() * 4, cudaMemcpyHostToDevice) == cudaSuccess &&
              cudaMemcpy(upa, L.up_arc.data(), L.up_arc.size() * 8, cudaMemcpyHostToDevice) == cudaSuccess &&
              cudaMemcpy(tb, h->tail_bits.data(), nw * 4, cudaMemcpyHostToDevice) == cudaSuccess &&
              cudaMemset(g.flags, 0, nw * 4) == cudaSuccess && cudaMemset(g.err, 0, 4) == cudaSuccess &&
              cudaMemset(g.seed_cnt, 0, SEED_SLOTS * KMAX * 4) == cudaSuccess &&
              cudaStreamCreateWithFlags(&h->side, cudaStreamNonBlocking) == cudaSuccess &&
              cudaDeviceSynchronize() == cudaSuccess;
    for (uint32_t s = 0; ok && s < SEED_SLOTS; s++)
        ok = cudaEventCreateWithFlags(&h->up_done[s], cudaEventDisableTiming) == cudaSuccess &&
             cudaEventCreateWithFlags(&h->slot_free[s], cudaEventDisableTiming) == cudaSuccess;
    if (!ok) { cudaGetLastError(); free_device(h); return PHAST_ECUDA; }
    return PHAST_OK;
}

int validate_csr(uint32_t n, const uint64_t* first, const uint32_t* head, const uint32_t* len) {
    if (n == 0 || n == 0xFFFFFFFFu || !first) return PHAST_EINVAL;
    if (first[0] != 0) return PHAST_EINVAL;
    for (uint32_t v = 0; v < n; v++)
        if (first[v + 1] < first[v]) return PHAST_EINVAL;
    uint64_t m = first[n];
    if (m && (!head || !len)) return PHAST_EINVAL;
    for (uint64_t e = 0; e < m; e++)
        if (head[e] >= n) return PHAST_EINVAL;
    return PHAST_OK;
}

int map_sources(const phast_ctx* h, const uint32_t* src, uint32_t k, Sources& S) {
    for (uint32_t i = 0; i < k; i++) {
        if (src[i] >= h->n) return PHAST_ERANGE;
        S.s[i] = h->L.perm[src[i]];
    }
    for (uint32_t i = k; i < KMAX; i++) S.s[i] = 0;
    return PHAST_OK;
}

// Chunk size: at most sweep_chunk_vertices(k); in the wavefront layout small enough
// that one iteration of all CTAs (grid * cap vertices) stays under delta / 2, so that
// almost every dependency points at least one iteration back (few pad slots).
uint32_t chunk_cap_for(const Layout& L, uint32_t k, uint32_t grid) {
    const uint32_t vmax = sweep_chunk_vertices(k), vpp = sweep_pass_vertices(k);
    if (L.mode != LAYOUT_WAVEFRONT) return vmax;
    uint32_t cap = L.delta / (2 * std::max(1u, grid));
    cap = cap / vpp * vpp;
    return std::max(vpp, std::min(vmax, cap));
}

// Plan of the persistent sweep for one k.  Chunks are contiguous internal-id ranges
// of at most CV vertices, cut wherever a vertex has a G-down tail inside the open
// chunk (so a chunk never waits on itself).  Chunk c is processed by CTA c % grid in
// iteration c / grid; it depends on the iteration of the latest chunk holding one
// of its tails, and may start once every CTA has finished that iteration.
phast_ctx::Plan* get_plan(phast_ctx* h, uint32_t k) {
    auto it = h->plans.find(k);
    if (it != h->plans.end()) return it->second.ok ? &it->second : nullptr;
    phast_ctx::Plan& P = h->plans[k];
    const Layout& L = h->L;
    SweepPlan& p = P.p;
    p.k = k;
    p.variant = h->sweep_mode == 2 ? 0u : h->sweep_mode == 3 ? 1u : h->sweep_mode == 4 && k >= 4 ? 3u
              : h->sweep_mode == 5 ? 2u : h->sweep_mode == 6 ? 5u : h->sweep_mode == 7 ? 6u : 4u;
    uint32_t nseg_top = 0, seg_from = 0;
    const char* bseg = std::getenv("PHAST_BOTTOM_SEG");
    if (h->sweep_mode == 1 && L.mode == LAYOUT_DIAGONAL && bseg && std::atoi(bseg)) {
        // the diagonals of the bottom levels in ONE launch; segment j waits only for
        // segment j - lag (the layout's guarantee), the top levels stay one launch each
        seg_from = L.levels - L.cut;
        P.bottom_from = seg_from;
        p.variant = 6;
    } else if (h->sweep_mode == 1) {   // hybrid: the small top segments as one segment-barrier launch, big ones one launch each
        uint32_t thresh = 0;
        if (const char* e = std::getenv("PHAST_TOP_THRESH")) thresh = (uint32_t)std::atoi(e);
        uint32_t J = 0;
        while (J + 1 < L.lvl_off.size() && L.lvl_off[J + 1] - L.lvl_off[J] < thresh) J++;
        if (J < 2) return nullptr;           // nothing worth fusing
        P.top_levels = J;
        nseg_top = J;
        p.variant = 6;
    }
    int occ = std::min(sweep_blocks_per_sm(k, false, p.variant), sweep_blocks_per_sm(k, true, p.variant));
    p.grid = (uint32_t)std::max(1, occ * num_sms());
    p.err = h->g.err;
    if (p.variant == 6) {   // segment barriers: the segments of the layout, one grid barrier between two
        if ((uint64_t)h->n * 16 >= 0x7FFFFFFFull) return nullptr;   // 32-bit item indices
        // CTAs per SM: all (8) for a whole sweep; for the hybrid's top levels fewer, so
        // that the next batch's upward searches (side stream) stay co-resident and never
        // hold back a CTA of this grid (every CTA must be resident for the barriers)
        int per_sm = nseg_top ? 4 : 8;
        if (const char* e = std::getenv(nseg_top ? "PHAST_TOP_CTAS" : "PHAST_SEG_CTAS")) per_sm = std::max(1, std::atoi(e));
        p.grid = (uint32_t)std::max(1, std::min(occ, per_sm) * num_sms());
        const uint32_t nseg = nseg_top ? nseg_top : (uint32_t)L.lvl_off.size() - 1 - seg_from;
        p.nchunks = p.iters = nseg;
        p.chunk_cap = seg_from ? 0u : L.mode == LAYOUT_DIAGONAL ? L.levels - L.cut : nseg;   // diagonals: by tail bit
        p.stream_last = nseg_top ? 0u : 1u;   // the layout's last segment is nobody's tail
        p.seg_lag = seg_from ? L.lag : 1u;
        uint32_t *a, *w;
        if (dmalloc(&a, nseg + 1) || dmalloc(&w, nseg)) return nullptr;
        p.chunk_v = a;
        p.wave_done = w;
        if (cudaMemcpy(a, L.lvl_off.data() + seg_from, (size_t)(nseg + 1) * 4, cudaMemcpyHostToDevice) != cudaSuccess ||
            cudaMemset(w, 0, (size_t)nseg * 4) != cudaSuccess) {
            cudaGetLastError();
            return nullptr;
        }
        P.ok = true;
        return &P;
    }
    if (p.variant == 5) {   // warp waves: one wave = one chunk of every warp (layout.cpp: plan_waves)
        p.workers = p.grid * SWEEP_WARPS;
        uint32_t window = 4;
        if (const char* e = std::getenv("PHAST_WAVE_WINDOW")) window = (uint32_t)std::atoi(e);
        WavePlan wp;
        if (plan_waves(L, sweep_wave_chunk_vertices(k), sweep_wave_chunk_arcs(), p.workers, window, wp))
            return nullptr;
        p.nchunks = wp.chunks;
        p.iters = wp.waves;
        p.chunk_cap = (wp.waves + 63) / 64 * 64;   // sub-counter stride: each sub-counter array on its own lines
        if (std::getenv("PHAST_VERBOSE"))
            std::fprintf(stderr, "wave plan k=%u: T=%u chunks=%u waves=%u pads=%u lag1=%llu lag2=%llu lag3=%llu lag4+=%llu\n",
                         k, p.workers, wp.chunks, wp.waves, wp.pads, (unsigned long long)wp.lag_hist[0],
                         (unsigned long long)wp.lag_hist[1], (unsigned long long)wp.lag_hist[2],
                         (unsigned long long)wp.lag_hist[3]);
        uint32_t *a, *w;
        const size_t nc = (size_t)sweep_wave_subcounters() * p.chunk_cap;
        if (dmalloc(&a, wp.desc.size() + 4) || dmalloc(&w, nc)) return nullptr;
        p.wdesc = reinterpret_cast<const uint4*>(a);
        p.wave_done = w;
        if ((!wp.desc.empty() && cudaMemcpy(a, wp.desc.data(), wp.desc.size() * 4, cudaMemcpyHostToDevice) != cudaSuccess) ||
            cudaMemset(w, 0, nc * 4) != cudaSuccess) {
            cudaGetLastError();
            return nullptr;
        }
        P.ok = true;
        return &P;
    }
    if (p.variant == 2 || p.variant == 4) {
        p.workers = p.grid * (SWEEP_WARPS);
        WarpPlan wp;
        const uint32_t cap = p.variant == 4 ? sweep_wpipe_chunk_vertices(k) : sweep_warp_chunk_vertices(k);
        if (plan_warp_chunks(L, cap, p.workers, wp, p.variant == 4 ? 126u : 0u)) return nullptr;
        p.nchunks = wp.chunks;
        p.chunk_cap = cap;
        if (p.variant == 4) {   // per-chunk {vbeg, vend, e0, e1} for the cp.async staging
            std::vector<uint32_t> info((size_t)wp.chunks * 4);
            for (uint32_t j = 0; j < wp.chunks; j++) {
                const uint32_t vb = wp.meta[4 * (size_t)j], ve = wp.meta[4 * (size_t)j + 1];
                info[4 * (size_t)j + 0] = vb;
                info[4 * (size_t)j + 1] = ve;
                info[4 * (size_t)j + 2] = L.dn_first[vb];
                info[4 * (size_t)j + 3] = L.dn_first[ve];
            }
            uint32_t* pi;
            if (dmalloc(&pi, info.size())) return nullptr;
            p.pinfo = reinterpret_cast<const uint4*>(pi);
            if (cudaMemcpy(pi, info.data(), info.size() * 4, cudaMemcpyHostToDevice) != cudaSuccess) {
                cudaGetLastError();
                return nullptr;
            }
        }
        uint32_t *a, *b, *w;
        if (dmalloc(&a, wp.meta.size()) || dmalloc(&b, wp.deps.size()) || dmalloc(&w, wp.chunks)) return nullptr;
        p.wmeta = reinterpret_cast<const uint4*>(a); p.wdeps = b; p.done = w;
        if (cudaMemcpy(a, wp.meta.data(), wp.meta.size() * 4, cudaMemcpyHostToDevice) != cudaSuccess ||
            (!wp.deps.empty() &&
             cudaMemcpy(b, wp.deps.data(), wp.deps.size() * 4, cudaMemcpyHostToDevice) != cudaSuccess) ||
            cudaMemset(w, 0, (size_t)wp.chunks * 4) != cudaSuccess) {
            cudaGetLastError();
            return nullptr;
        }
        P.ok = true;
        return &P;
    }
    if (p.variant == 3) {   // pipelined gather: CTA chunks, per-chunk completion flags, one-chunk lookahead
        uint32_t gv = 0, cap_arcs = 0;
        sweep_pipe_geometry(k, &gv, &cap_arcs);
        p.workers = p.grid;
        p.chunk_cap = gv;
        WarpPlan wp;
        if (plan_warp_chunks(L, gv, p.workers, wp, cap_arcs)) return nullptr;
        p.nchunks = wp.chunks;
        std::vector<uint32_t> info((size_t)wp.chunks * 4);
        for (uint32_t j = 0; j < wp.chunks; j++) {
            const uint32_t vb = wp.meta[4 * (size_t)j], ve = wp.meta[4 * (size_t)j + 1];
            info[4 * (size_t)j + 0] = vb;
            info[4 * (size_t)j + 1] = ve;
            info[4 * (size_t)j + 2] = L.dn_first[vb];
            info[4 * (size_t)j + 3] = L.dn_first[ve];
        }
        uint32_t *a, *b, *w, *pi;
        if (dmalloc(&a, wp.meta.size()) || dmalloc(&b, wp.deps.size()) || dmalloc(&w, wp.chunks) ||
            dmalloc(&pi, info.size()))
            return nullptr;
        p.wmeta = reinterpret_cast<const uint4*>(a); p.wdeps = b; p.done = w;
        p.pinfo = reinterpret_cast<const uint4*>(pi);
        if (cudaMemcpy(a, wp.meta.data(), wp.meta.size() * 4, cudaMemcpyHostToDevice) != cudaSuccess ||
            (!wp.deps.empty() &&
             cudaMemcpy(b, wp.deps.data(), wp.deps.size() * 4, cudaMemcpyHostToDevice) != cudaSuccess) ||
            cudaMemcpy(pi, info.data(), info.size() * 4, cudaMemcpyHostToDevice) != cudaSuccess ||
            cudaMemset(w, 0, (size_t)wp.chunks * 4) != cudaSuccess) {
            cudaGetLastError();
            return nullptr;
        }
        P.ok = true;
        return &P;
    }
    const uint32_t CV = chunk_cap_for(h->L, k, p.grid);
    p.chunk_cap = CV;
    ChunkPlan cp;
    if (plan_chunks(L, CV, p.grid, cp, 0, 1, 0)) return nullptr;
    p.nchunks = cp.slots;
    p.iters = (cp.slots + p.grid - 1) / p.grid;
    const std::vector<uint32_t>& cv = cp.slot_v;
    const std::vector<uint32_t>& dep = cp.dep;
    uint32_t *a, *b, *w;
    if (dmalloc(&a, cv.size()) || dmalloc(&b, dep.size()) || dmalloc(&w, p.iters)) return nullptr;
    p.chunk_v = a; p.chunk_dep = b; p.wave_done = w;
    if (cudaMemcpy(a, cv.data(), cv.size() * 4, cudaMemcpyHostToDevice) != cudaSuccess ||
        cudaMemcpy(b, dep.data(), dep.size() * 4, cudaMemcpyHostToDevice) != cudaSuccess ||
        cudaMemset(w, 0, (size_t)p.iters * 4) != cudaSuccess) {
        cudaGetLastError();
        return nullptr;
    }
    P.ok = true;
    return &P;
}

// Chunks of one segment [a, b) over a CSR (offsets `f`): <= VCH vertices and <= ECH
// arcs each; chunks without arcs change nothing and are skipped.
void push_chunks(std::vector<uint4>& ch, const uint32_t* f, uint32_t a, uint32_t b, bool big) {
    const uint32_t VCH = top_chunk_vertices(big), ECH = top_chunk_arcs(big);
    uint32_t v = a;
    while (v < b) {
        uint32_t w = v;
        while (w < b && w - v < VCH && f[w + 1] - f[v] <= ECH) w++;
        bool heavy = false;
        for (uint32_t x = v; x < w; x++) heavy |= f[x + 1] - f[x] > top_heavy_arcs();
        if (f[w] > f[v]) ch.push_back(make_uint4(v, w | (heavy ? 0x80000000u : 0u), f[v], f[w]));
        v = w;
    }
}

// A-up in-arcs by head, uploaded once (graphs small enough for a fused query).
bool ensure_upin(phast_ctx* h) {
    if (h->d_upin_first) return true;
    if (h->upin_tried) return false;
    h->upin_tried = true;
    const Layout& L = h->L;
    const uint32_t n = h->n;
    std::vector<uint32_t> f((size_t)n + 1, 0);
    for (const Arc& a : L.up_arc) f[a.x + 1]++;
    for (uint32_t v = 0; v < n; v++) f[v + 1] += f[v];
    std::vector<Arc> arc(L.up_arc.size());
    std::vector<uint32_t> pos(f.begin(), f.end() - 1);
    for (uint32_t u = 0; u < n; u++)
        for (uint32_t e = L.up_first[u]; e < L.up_first[u + 1]; e++) arc[pos[L.up_arc[e].x]++] = Arc{u, L.up_arc[e].y};
    for (uint32_t v = 0; v < n; v++)
        if (f[v + 1] - f[v] > top_chunk_arcs(true)) return false;
    uint32_t* df = nullptr;
    uint2* da = nullptr;
    // +4 / +2 elements: the 16-byte aligned bulk copies may read past the end
    if (dmalloc(&df, f.size() + 4) || dmalloc(&da, arc.size() + 2)) {
        cudaFree(df);
        return false;
    }
    if (cudaMemset(df, 0, (f.size() + 4) * 4) != cudaSuccess || cudaMemset(da, 0, (arc.size() + 2) * 8) != cudaSuccess ||
        cudaMemcpy(df, f.data(), f.size() * 4, cudaMemcpyHostToDevice) != cudaSuccess ||
        (!arc.empty() && cudaMemcpy(da, arc.data(), arc.size() * 8, cudaMemcpyHostToDevice) != cudaSuccess)) {
        cudaGetLastError();
        cudaFree(df);
        cudaFree(da);
        return false;
    }
    h->d_upin_first = df;
    h->d_upin_arc = da;
    return true;
}

// Shared-memory sweep plans (kernels.cu: sweep_top_kernel), one per k:
//  - fused: the whole graph's rows fit the label budget -> the whole query (G-up
//    pull sweep, then the G-down sweep) in one launch.  PHAST_FUSED=0 disables it;
//  - top: the longest prefix of levels whose rows [0, V) fit, each level small
//    enough for one SM (<= 32 items per consumer thread); the rest one launch per
//    level.  PHAST_TOP=0 disables it; PHAST_TOP_MAXV caps V.
// Both need every vertex to have at most top_chunk_arcs(big) in-arcs; big chunks
// (top_big_fits) when the rows leave room for them.
phast_ctx::Top* get_top(phast_ctx* h, uint32_t k) {
    auto it = h->tops.find(k);
    if (it != h->tops.end()) return it->second.ok ? &it->second : nullptr;
    phast_ctx::Top& T = h->tops[k];
    const Layout& L = h->L;
    if (L.mode != LAYOUT_LEVELS && L.mode != LAYOUT_LEVELS_BFS) return nullptr;
    if (L.lvl_off.size() < 2 || h->n >= 0x80000000u) return nullptr;   // chunk vend carries a flag bit
    const uint32_t nseg = (uint32_t)L.lvl_off.size() - 1;
    const uint32_t G = k >= 4 ? k / 4 : 1;
    const uint32_t ECH = top_chunk_arcs(false);
    const uint64_t vmax_budget = top_label_budget() / (4ull * k);
    std::vector<uint4> ch;
    const char* fe = std::getenv("PHAST_FUSED");
    bool fused = !(fe && std::atoi(fe) == 0) && h->n <= vmax_budget;
    const bool fbig = fused && top_big_fits(k, h->n);
    const uint32_t ECHf = top_chunk_arcs(fbig);
    for (uint32_t v = 0; fused && v < h->n; v++) fused = L.dn_first[v + 1] - L.dn_first[v] <= ECHf;
    std::vector<uint32_t> f;
    if (fused && ensure_upin(h)) {
        f.resize((size_t)h->n + 1);
        if (cudaMemcpy(f.data(), h->d_upin_first, f.size() * 4, cudaMemcpyDeviceToHost) != cudaSuccess) {
            cudaGetLastError();
            return nullptr;
        }
        for (uint32_t v = 0; fused && v < h->n; v++) fused = f[v + 1] - f[v] <= ECHf;
    } else {
        fused = false;
    }
    if (fused) {
        for (uint32_t j = nseg; j-- > 0;) push_chunks(ch, f.data(), L.lvl_off[j], L.lvl_off[j + 1], fbig);   // ascending levels
        T.a.split = (uint32_t)ch.size();
        for (uint32_t j = 0; j < nseg; j++) push_chunks(ch, L.dn_first.data(), L.lvl_off[j], L.lvl_off[j + 1], fbig);
        T.a.big = fbig;
        T.a.first[0] = h->d_upin_first;
        T.a.arcs[0] = h->d_upin_arc;
        T.a.fused = 1;
        T.J = T.J2 = nseg;
        T.a.V = h->n;
    } else {
        const char* env = std::getenv("PHAST_TOP");   // PHAST_TOP=0: no shared-memory top launch
        uint64_t vmax = vmax_budget;
        if (const char* e = std::getenv("PHAST_TOP_MAXV")) vmax = std::min<uint64_t>(vmax, (uint64_t)std::atoll(e));
        uint32_t J = 0;
        while (J < nseg) {
            const uint32_t a = L.lvl_off[J], b = L.lvl_off[J + 1];
            if (b > vmax || (uint64_t)(b - a) * G > 32ull * 992) break;
            bool fits = true;
            for (uint32_t v = a; v < b && fits; v++) fits = L.dn_first[v + 1] - L.dn_first[v] <= ECH;
            if (!fits) break;
            J++;
        }
        if (J < 2 || (env && std::atoi(env) == 0)) J = 0;
        // hybrid upward search (PHAST_UP_HYBRID=0 disables): the upward kernel expands
        // only vertices below the top levels; the top kernel finishes G-up inside
        // [0, V) with a pull pass in ascending level order (reading R9), then sweeps
        // G-down.  Exact: a G-up path only climbs, so it enters [0, V) once and its part
        // below V is found by the search, its part inside by the pull pass.
        // When: the upward searches run beside the previous batch's sweep (side stream),
        // so moving work from them into the top kernel only pays when they are the
        // critical path, i.e. when a sweep is shorter than the searches: estimated sweep
        // 8kn B at ~5 TB/s vs ~2 us per search wave (<= one per level).  Measured (r43):
        // C2 k=16 14.1 vs 14.9 us/tree, C2D 50.9 vs 61.5 (hybrid); C2 k=64 3.87 vs 3.60,
        // C3 k=64 2.069 vs 2.058 ms/step (full searches).  PHAST_UP_HYBRID=0/1 forces it.
        const char* he = std::getenv("PHAST_UP_HYBRID");
        const uint32_t V = L.lvl_off[J];
        const bool big = J && top_big_fits(k, V);
        T.a.big = big;
        const double sweep_us = 8.0 * k * h->n / 5e6, search_us = 2.0 * L.levels;
        const bool hybrid = he ? std::atoi(he) != 0 : sweep_us < search_us;
        if (J && hybrid) {
            std::vector<uint32_t> f((size_t)V + 1, 0);
            for (uint32_t u = 0; u < V; u++)
                for (uint32_t e = L.up_first[u]; e < L.up_first[u + 1]; e++) f[L.up_arc[e].x + 1]++;
            for (uint32_t v = 0; v < V; v++) f[v + 1] += f[v];
            std::vector<Arc> arc(f[V]);
            std::vector<uint32_t> pos(f.begin(), f.end() - 1);
            for (uint32_t u = 0; u < V; u++)
                for (uint32_t e = L.up_first[u]; e < L.up_first[u + 1]; e++)
                    arc[pos[L.up_arc[e].x]++] = Arc{u, L.up_arc[e].y};
            bool fits = true;
            for (uint32_t v = 0; v < V && fits; v++) fits = f[v + 1] - f[v] <= top_chunk_arcs(big);
            if (fits && !dmalloc(&T.up_f, f.size() + 4) && !dmalloc(&T.up_a, arc.size() + 2) &&
                cudaMemset(T.up_f, 0, (f.size() + 4) * 4) == cudaSuccess &&
                cudaMemset(T.up_a, 0, (arc.size() + 2) * 8) == cudaSuccess &&
                cudaMemcpy(T.up_f, f.data(), f.size() * 4, cudaMemcpyHostToDevice) == cudaSuccess &&
                (arc.empty() || cudaMemcpy(T.up_a, arc.data(), arc.size() * 8, cudaMemcpyHostToDevice) == cudaSuccess)) {
                for (uint32_t j = J; j-- > 0;) push_chunks(ch, f.data(), L.lvl_off[j], L.lvl_off[j + 1], big);
                T.a.first[0] = T.up_f;
                T.a.arcs[0] = T.up_a;
                T.vtop = V;
            } else {
                cudaGetLastError();
            }
        }
        T.a.split = (uint32_t)ch.size();
        for (uint32_t j = 0; j < J; j++) push_chunks(ch, L.dn_first.data(), L.lvl_off[j], L.lvl_off[j + 1], big);
        T.J = J;
        T.a.V = V;
        // the next levels, while small, in one cluster launch (PHAST_CL_SIZE=0 disables;
        // PHAST_CL_PASSES: max grid-stride passes of the cluster per level, default 8)
        uint32_t J2 = J;
        const uint64_t CT = cluster_threads();
        uint64_t passes = 8;
        if (const char* e = std::getenv("PHAST_CL_PASSES")) passes = (uint64_t)std::max(1, std::atoi(e));
        if (CT && h->g.dn_rec)
            while (J2 + 1 < nseg && (uint64_t)(L.lvl_off[J2 + 1] - L.lvl_off[J2]) * G <= CT * passes) J2++;
        if (J2 - J < 2) J2 = J;   // not worth a launch
        if (J == 0 && J2 == 0) return nullptr;
        if (J2 > J) {
            if (dmalloc(&T.cl_seg, J2 - J + 1) ||
                cudaMemcpy(T.cl_seg, L.lvl_off.data() + J, (size_t)(J2 - J + 1) * 4, cudaMemcpyHostToDevice) !=
                    cudaSuccess) {
                cudaGetLastError();
                return nullptr;
            }
        }
        T.J2 = J2;
    }
    const bool none = ch.empty();
    if (none) ch.push_back(make_uint4(0, 0, 0, 0));   // keep a valid device array
    if (dmalloc(&T.chunks, ch.size()) ||
        cudaMemcpy(T.chunks, ch.data(), ch.size() * sizeof(uint4), cudaMemcpyHostToDevice) != cudaSuccess) {
        cudaGetLastError();
        return nullptr;
    }
    T.a.chunks = T.chunks;
    T.a.nchunks = none ? 0u : (uint32_t)ch.size();
    T.a.first[1] = h->g.dn_first;
    T.a.arcs[1] = h->g.dn_arc;
    T.ok = true;
    if (std::getenv("PHAST_VERBOSE"))
        std::fprintf(stderr, "%s plan k=%u: %u levels, %u vertices, %u chunks (%u up); cluster levels [%u, %u)\n",
                     T.a.fused ? "fused" : "top", k, T.J, T.a.V, T.a.nchunks, T.a.split, T.J, T.J2);
    return &T;
}

constexpr size_t MAX_TIMED_BATCHES = 16384;

cudaEvent_t timing_event(phast_ctx* h) {
    if (h->ev_used >= 3 * MAX_TIMED_BATCHES) return nullptr;
    if (h->ev_used == h->ev.size()) {
        cudaEvent_t e;
        if (cudaEventCreate(&e) != cudaSuccess) { cudaGetLastError(); return nullptr; }
        h->ev.push_back(e);
    }
    return h->ev[h->ev_used++];
}

// one full query (a1-a3) for k mapped sources; diam != nullptr: fused max, rows of
// vertices that are nobody's tail are not stored
int run_query(phast_ctx* h, const Sources& S, uint32_t k, uint32_t* dist, uint32_t* diam, cudaStream_t st) {
    cudaEvent_t e0 = nullptr, e1 = nullptr, e2 = nullptr;
    if (h->timing && h->ev_used + 3 <= 3 * MAX_TIMED_BATCHES) {
        e0 = timing_event(h); e1 = timing_event(h); e2 = timing_event(h);
        if (!e0 || !e1 || !e2) return PHAST_ECUDA;
        cudaEventRecord(e0, st);
    }
    phast_ctx::Top* top = get_top(h, k);
    if (top && top->a.fused) {   // small graph: the whole query (a1-a3, a5) in one launch
        if (launch_sweep_top(top->a, k, S, dist, h->g.flags, diam, st) != cudaSuccess) return PHAST_ECUDA;
        if (e1) cudaEventRecord(e1, st);   // no separate upward stage: all of it counts as the sweep
        if (e2) cudaEventRecord(e2, st);
        return PHAST_OK;
    }
    // a1 on the side stream (overlaps the previous batch's sweep), a2 on the caller's stream
    const uint32_t slot = h->slot_next;
    h->slot_next = (h->slot_next + 1) % SEED_SLOTS;
    if (cudaStreamWaitEvent(h->side, h->slot_free[slot], 0) != cudaSuccess) return PHAST_ECUDA;
    phast_ctx::Plan* plan = get_plan(h, k);
    // the top / cluster launches run only on the per-level path (no persistent plan)
    if (plan || h->L.mode == LAYOUT_DIAGONAL || h->L.lvl_off.empty()) top = nullptr;
    const uint32_t vtop = (top && top->J) ? top->vtop : 0u;
    if (launch_upward(h->g, S, k, slot, vtop, h->side) != cudaSuccess) return PHAST_ECUDA;
    if (cudaEventRecord(h->up_done[slot], h->side) != cudaSuccess) return PHAST_ECUDA;
    if (cudaStreamWaitEvent(st, h->up_done[slot], 0) != cudaSuccess) return PHAST_ECUDA;
    if (launch_seed(h->g, k, slot, dist, st) != cudaSuccess) return PHAST_ECUDA;
    if (e1) cudaEventRecord(e1, st);
    if (plan && plan->bottom_from) {   // top levels one launch each, then the bottom diagonals in one launch
        for (uint32_t j = 0; j < plan->bottom_from; j++)
            if (launch_sweep_level(h->g, k, h->L.lvl_off[j], h->L.lvl_off[j + 1], dist, diam, true, false, false,
                                   st) != cudaSuccess)
                return PHAST_ECUDA;
        if ((uint64_t)(plan->epoch + 1) * plan->p.grid >= 0x7FFFFFFFull) {
            if (cudaMemsetAsync(plan->p.wave_done, 0, (size_t)plan->p.iters * 4, st) != cudaSuccess) return PHAST_ECUDA;
            plan->epoch = 0;
        }
        plan->epoch++;
        if (launch_sweep_persistent(h->g, plan->p, plan->epoch, dist, diam, st) != cudaSuccess) return PHAST_ECUDA;
    } else if (plan && plan->top_levels == 0) {   // a3 + a4: one persistent launch, dataflow over chunks
        if ((plan->p.variant < 2 || plan->p.variant == 6) && (uint64_t)(plan->epoch + 1) * plan->p.grid >= 0x7FFFFFFFull) {
            if (cudaMemsetAsync(plan->p.wave_done, 0, (size_t)plan->p.iters * 4, st) != cudaSuccess) return PHAST_ECUDA;
            plan->epoch = 0;
        }
        if (plan->p.variant == 5 &&
            (uint64_t)(plan->epoch + 1) * (plan->p.workers / sweep_wave_subcounters()) >= 0x7FFFFFFFull) {
            if (cudaMemsetAsync(plan->p.wave_done, 0,
                                (size_t)sweep_wave_subcounters() * plan->p.chunk_cap * 4, st) != cudaSuccess)
                return PHAST_ECUDA;
            plan->epoch = 0;
        }
        plan->epoch++;
        if (launch_sweep_persistent(h->g, plan->p, plan->epoch, dist, diam, st) != cudaSuccess) return PHAST_ECUDA;
    } else if (!h->L.lvl_off.empty()) {   // one launch per level (§VI), level layout only
        const uint32_t levels = (uint32_t)h->L.lvl_off.size() - 1;   // segments
        const bool diagonal = h->L.mode == LAYOUT_DIAGONAL;
        uint32_t j0 = 0;
        if (top) {                            // the small top levels in one single-CTA launch,
            if (top->J && launch_sweep_top(top->a, k, S, dist, h->g.flags, diam, st) != cudaSuccess)
                return PHAST_ECUDA;
            if (top->J2 > top->J &&           // the next small ones in one cluster launch
                launch_sweep_cluster(h->g, k, top->cl_seg, top->J2 - top->J, dist, diam, st) != cudaSuccess)
                return PHAST_ECUDA;
            j0 = top->J2;
        } else if (plan) {                    // hybrid: small top levels in one persistent launch
            if ((uint64_t)(plan->epoch + 1) * plan->p.grid >= 0x7FFFFFFFull) {
                if (cudaMemsetAsync(plan->p.wave_done, 0, (size_t)plan->p.iters * 4, st) != cudaSuccess)
                    return PHAST_ECUDA;
                plan->epoch = 0;
            }
            plan->epoch++;
            if (launch_sweep_persistent(h->g, plan->p, plan->epoch, dist, diam, st) != cudaSuccess)
                return PHAST_ECUDA;
            j0 = plan->top_levels;
        }
        for (uint32_t j = j0; j < levels; j++) {
            bool last = (j + 1 == levels);
            bool store = !(diam && last);   // level-0 rows are never read again (diameter mode)
            const bool by_tail = diagonal && j >= h->L.levels - h->L.cut;   // diagonals mix levels
            if (launch_sweep_level(h->g, k, h->L.lvl_off[j], h->L.lvl_off[j + 1], dist, diam, store, last, by_tail,
                                   st) !=
                cudaSuccess)
                return PHAST_ECUDA;
        }
    } else {
        return PHAST_EINTERNAL;
    }
    if (launch_clear_flags(h->g, k, slot, st) != cudaSuccess) return PHAST_ECUDA;
    if (cudaEventRecord(h->slot_free[slot], st) != cudaSuccess) return PHAST_ECUDA;   // seeds of `slot` consumed
    if (e2) cudaEventRecord(e2, st);
    return PHAST_OK;
}

ChOptions to_ch_options(const phast_opts* o) {
    ChOptions c;
    if (o) {
        if (o->hop_limit_lo) c.hop_limit_lo = o->hop_limit_lo;
        if (o->hop_limit_hi) c.hop_limit_hi = o->hop_limit_hi;
        if (o->settled_cap) c.settled_cap = o->settled_cap;
        c.threads = o->threads;
    }
    return c;
}

int ensure_in_csr(phast_ctx* h) {
    int rc;
    if (!h->d_in_first) {   // upload the original in-CSR on first use (parents, betweenness)
        uint32_t* f = nullptr;
        uint2* a = nullptr;
        if ((rc = dmalloc(&f, h->L.in_first.size())) || (rc = dmalloc(&a, h->L.in_arc.size() + 1))) {
            cudaFree(f);
            return rc;
        }
        if (cudaMemcpy(f, h->L.in_first.data(), h->L.in_first.size() * 4, cudaMemcpyHostToDevice) != cudaSuccess ||
            (!h->L.in_arc.empty() &&
             cudaMemcpy(a, h->L.in_arc.data(), h->L.in_arc.size() * 8, cudaMemcpyHostToDevice) != cudaSuccess)) {
            cudaGetLastError();
            cudaFree(f);
            cudaFree(a);
            return PHAST_ECUDA;
        }
        h->d_in_first = f;
        h->d_in_arc = a;
    }
    return PHAST_OK;
}

// Original out-arcs by tail {head, len} in internal ids: the transpose of L.in_arc
// (betweenness delta pass), uploaded on first use.
int ensure_out_csr(phast_ctx* h) {
    if (h->d_out_first) return PHAST_OK;
    const uint32_t n = h->n;
    const auto& F = h->L.in_first;
    const auto& A = h->L.in_arc;
    std::vector<uint32_t> of(n + 1, 0);
    for (const auto& a : A) of[a.x + 1]++;
    for (uint32_t v = 0; v < n; v++) of[v + 1] += of[v];
    std::vector<uint32_t> fill(of.begin(), of.end() - 1);
    std::vector<Arc> oa(A.size());
    for (uint32_t w = 0; w < n; w++)
        for (uint32_t e = F[w]; e < F[w + 1]; e++) oa[fill[A[e].x]++] = Arc{w, A[e].y};
    uint32_t* f = nullptr;
    uint2* a = nullptr;
    int rc;
    if ((rc = dmalloc(&f, of.size())) || (rc = dmalloc(&a, oa.size() + 1))) {
        cudaFree(f);
        return rc;
    }
    if (cudaMemcpy(f, of.data(), of.size() * 4, cudaMemcpyHostToDevice) != cudaSuccess ||
        (!oa.empty() && cudaMemcpy(a, oa.data(), oa.size() * 8, cudaMemcpyHostToDevice) != cudaSuccess)) {
        cudaGetLastError();
        cudaFree(f);
        cudaFree(a);
        return PHAST_ECUDA;
    }
    h->d_out_first = f;
    h->d_out_arc = a;
    return PHAST_OK;
}

int ensure_scratch(phast_ctx* h, size_t elems) {
    if (h->dist_scratch_elems >= elems) return PHAST_OK;
    cudaFree(h->dist_scratch);
    h->dist_scratch = nullptr;
    h->dist_scratch_elems = 0;
    int rc = dmalloc(&h->dist_scratch, elems);
    if (rc) return rc;
    h->dist_scratch_elems = elems;
    return PHAST_OK;
}

}  // namespace

extern "C" {

int phast_build(uint32_t n, const uint64_t* first, const uint32_t* head, const uint32_t* len, const phast_opts* opts,
                phast_ctx** out) {
    if (!out) return PHAST_EINVAL;
    *out = nullptr;
    int rc = validate_csr(n, first, head, len);
    if (rc) return rc;
    std::unique_ptr<phast_ctx> h(new (std::nothrow) phast_ctx());
    if (!h) return PHAST_ENOMEM;
    uint32_t flags = opts ? opts->flags : 0u;
    uint32_t delta = (opts && opts->delta) ? opts->delta : DEFAULT_DELTA;
    try {
        ChResult R;
        rc = ch_build(n, first, head, len, to_ch_options(opts), R);
        if (rc) return rc;
        h->n = n;
        h->m = first[n];
        h->shortcuts = R.shortcuts;
        h->rounds = R.rounds;
        const uint32_t mode = (flags & PHAST_FLAG_DIAGONAL)    ? LAYOUT_DIAGONAL
                              : (flags & PHAST_FLAG_WAVEFRONT) ? LAYOUT_WAVEFRONT
                              : ((flags & PHAST_FLAG_LEVEL_LAYOUT) && !(flags & PHAST_FLAG_BFS_IN_LEVEL))
                                  ? LAYOUT_LEVELS
                                  : LAYOUT_LEVELS_BFS;
        rc = layout_build(R, first, head, mode, delta, h->L);
        h->build_seconds = R.seconds;
        if (rc) return rc;
        rc = build_in_csr(h->L, n, first, head, len);
        if (rc) return rc;
        compute_tail_bits(h.get());
    } catch (const std::bad_alloc&) {
        return PHAST_ENOMEM;
    }
    if (!(flags & PHAST_FLAG_HOST_ONLY)) {
        rc = upload(h.get());
        if (rc) return rc;
    }
    *out = h.release();
    return PHAST_OK;
}

int phast_trees(phast_ctx* h, const uint32_t* sources, uint32_t k, uint32_t* dist, void* stream) {
    if (!h || !sources || !dist || !k_ok(k)) return PHAST_EINVAL;
    if (h->device < 0) return PHAST_ESTATE;
    if (k % 4 == 0 && ((uintptr_t)dist & 15)) return PHAST_EINVAL;
    Sources S;
    int rc = map_sources(h, sources, k, S);
    if (rc) return rc;
    DeviceGuard dg(h->device);
    if (!dg.ok) return PHAST_ECUDA;
    return run_query(h, S, k, dist, nullptr, (cudaStream_t)stream);
}

int phast_sync(phast_ctx* h, void* stream) {
    if (!h) return PHAST_EINVAL;
    if (h->device < 0) return PHAST_ESTATE;
    DeviceGuard dg(h->device);
    cudaError_t ce = cudaStreamSynchronize((cudaStream_t)stream);
    if (ce != cudaSuccess) {
        cudaGetLastError();
        if (std::getenv("PHAST_VERBOSE")) std::fprintf(stderr, "phast_sync: %s\n", cudaGetErrorString(ce));
        return PHAST_ECUDA;
    }
    uint32_t err = 0;
    if (cudaMemcpy(&err, h->g.err, 4, cudaMemcpyDeviceToHost) != cudaSuccess) return PHAST_ECUDA;
    if (err) {
        if (std::getenv("PHAST_VERBOSE")) std::fprintf(stderr, "phast_sync: device error word 0x%x\n", err);
        cudaMemset(h->g.err, 0, 4);
        return (err & 1u) ? PHAST_ERANGE : PHAST_ECUDA;   // bit 0: search-space overflow; bit 1: watchdog
    }
    return PHAST_OK;
}

int phast_trees_host(phast_ctx* h, const uint32_t* sources, uint32_t k, uint32_t* host_dist, void* stream) {
    if (!h || !sources || !host_dist || !k_ok(k)) return PHAST_EINVAL;
    if (h->device < 0) return PHAST_ESTATE;
    DeviceGuard dg(h->device);
    size_t elems = (size_t)h->n * k;
    int rc = ensure_scratch(h, elems);
    if (rc) return rc;
    rc = phast_trees(h, sources, k, h->dist_scratch, stream);
    if (rc) return rc;
    cudaStream_t st = (cudaStream_t)stream;
    if (cudaMemcpyAsync(host_dist, h->dist_scratch, elems * 4, cudaMemcpyDeviceToHost, st) != cudaSuccess)
        return PHAST_ECUDA;
    return phast_sync(h, stream);
}

int phast_parents(phast_ctx* h, const uint32_t* sources, uint32_t k, const uint32_t* dist, uint32_t* parent,
                  void* stream) {
    if (!h || !sources || !dist || !parent || !k_ok(k)) return PHAST_EINVAL;
    if (h->device < 0) return PHAST_ESTATE;
    if (k % 4 == 0 && (((uintptr_t)dist & 15) || ((uintptr_t)parent & 15))) return PHAST_EINVAL;
    if (h->L.in_first.size() != (size_t)h->n + 1) return PHAST_ESTATE;
    Sources S;
    int rc = map_sources(h, sources, k, S);
    if (rc) return rc;
    DeviceGuard dg(h->device);
    if ((rc = ensure_in_csr(h))) return rc;
    if (launch_parents(h->d_in_first, h->d_in_arc, h->n, S, k, dist, parent, (cudaStream_t)stream) != cudaSuccess)
        return PHAST_ECUDA;
    return PHAST_OK;
}

int phast_diameter(phast_ctx* h, const uint32_t* sources, uint64_t count, uint32_t k_batch, uint32_t* max_dev,
                   uint32_t* batch_max_dev, void* stream) {
    if (!h || !sources || !max_dev || count == 0 || !k_ok(k_batch)) return PHAST_EINVAL;
    if (h->device < 0) return PHAST_ESTATE;
    for (uint64_t i = 0; i < count; i++)
        if (sources[i] >= h->n) return PHAST_ERANGE;
    DeviceGuard dg(h->device);
    if (!dg.ok) return PHAST_ECUDA;
    cudaStream_t st = (cudaStream_t)stream;
    int rc = ensure_scratch(h, (size_t)h->n * k_batch);
    if (rc) return rc;
    uint64_t nb = (count + k_batch - 1) / k_batch;
    if (nb > 0xFFFFFFFFull) return PHAST_ERANGE;
    uint32_t* bm = batch_max_dev;
    if (!bm) {
        if (h->batch_max_elems < nb) {
            cudaFree(h->batch_max_scratch);
            h->batch_max_scratch = nullptr;
            h->batch_max_elems = 0;
            rc = dmalloc(&h->batch_max_scratch, nb);
            if (rc) return rc;
            h->batch_max_elems = nb;
        }
        bm = h->batch_max_scratch;
    }
    if (cudaMemsetAsync(bm, 0, nb * 4, st) != cudaSuccess) return PHAST_ECUDA;
    for (uint64_t b = 0; b < nb; b++) {
        Sources S;
        uint64_t base = b * k_batch;
        for (uint32_t i = 0; i < k_batch; i++) {
            uint64_t idx = base + i < count ? base + i : base;   // pad with a duplicate (max unchanged)
            S.s[i] = h->L.perm[sources[idx]];
        }
        rc = run_query(h, S, k_batch, h->dist_scratch, bm + b, st);
        if (rc) return rc;
    }
    if (launch_max_reduce(bm, (uint32_t)nb, max_dev, st) != cudaSuccess) return PHAST_ECUDA;
    return PHAST_OK;
}

}  // extern "C"

namespace {
// NEXT-3 driver shared by phast_betweenness (out = double cb[n]) and phast_reach
// (out = uint32 r[n]): per batch the trees, then the fixpoint(s), then the accumulation.
int centrality(phast_ctx* h, const uint32_t* sources, uint64_t count, uint32_t k_batch, void* out, bool reach,
               void* stream) {
    if (!h || !sources || !out || count == 0 || !k_ok(k_batch)) return PHAST_EINVAL;
    if (h->device < 0) return PHAST_ESTATE;
    if (h->L.in_first.size() != (size_t)h->n + 1) return PHAST_ESTATE;
    for (uint64_t i = 0; i < count; i++)
        if (sources[i] >= h->n) return PHAST_ERANGE;
    if (h->bc_len_ok == 0) {   // readings R16/R17: every original length > 0 (self-loops excepted)
        h->bc_len_ok = 1;
        for (const auto& a : h->L.in_arc)
            if (a.y == 0) h->bc_len_ok = -1;
    }
    if (h->bc_len_ok < 0) return PHAST_EINVAL;
    DeviceGuard dg(h->device);
    if (!dg.ok) return PHAST_ECUDA;
    cudaStream_t st = (cudaStream_t)stream;
    const uint32_t n = h->n, k = k_batch;
    const size_t elems = (size_t)n * k;
    if (elems >= 0xFFFFFFFFull) return PHAST_ERANGE;   // items are 32-bit
    int rc = ensure_scratch(h, elems);
    if (!rc) rc = ensure_in_csr(h);
    if (!rc) rc = ensure_out_csr(h);
    if (rc) return rc;
    constexpr uint32_t R = 30;   // passes per graph launch / host convergence check (multiple of 6)
    if (!h->bc_changed) {
        if ((rc = dmalloc(&h->bc_changed, R)) || (rc = dmalloc(&h->bc_qs, 3))) return rc;
        if (cudaMallocHost(&h->bc_changed_host, R * 4) != cudaSuccess) {
            cudaGetLastError();
            return PHAST_ENOMEM;
        }
    }
    if (h->bc_elems < elems) {
        cudaFree(h->bc_sigma);
        cudaFree(h->bc_delta);
        cudaFree(h->bc_q);
        h->bc_sigma = h->bc_delta = nullptr;
        h->bc_q = nullptr;
        h->bc_elems = 0;
        if ((rc = dmalloc(&h->bc_sigma, elems)) || (rc = dmalloc(&h->bc_delta, elems)) ||
            (rc = dmalloc(&h->bc_q, 3 * elems)))
            return rc;
        h->bc_elems = elems;
    }
    if (cudaMemsetAsync(out, 0, (size_t)n * (reach ? 4 : 8), st) != cudaSuccess) return PHAST_ECUDA;
    // Kahn order (kernels.cu): the count kernel fills queue 0; pass p reads queue p%2 with
    // size qs[p%3], appends to queue (p+1)%2 with qs[(p+1)%3], zeroes qs[(p+2)%3]; stop
    // after a pass that readied nothing (<= hop depth of the tight DAG + 1 passes)
    const BcGraph G{h->d_in_first, h->d_in_arc, h->d_out_first, h->d_out_arc};
    uint32_t* qbuf[2] = {h->bc_q, h->bc_q + elems};
    uint32_t* cnt = h->bc_q + 2 * elems;
    // R passes (+ clearing the change words before, reading them back after) are one CUDA
    // graph, captured once per call and direction on a private stream (the caller's stream
    // may be the legacy default stream, which cannot be captured); R is a multiple of 6,
    // so every chunk starts with the same queue/counter rotation.
    if ((!h->bc_ev && cudaEventCreateWithFlags(&h->bc_ev, cudaEventDisableTiming) != cudaSuccess) ||
        (!h->bc_stream && cudaStreamCreateWithFlags(&h->bc_stream, cudaStreamNonBlocking) != cudaSuccess)) {
        cudaGetLastError();
        return PHAST_ECUDA;
    }
    cudaStream_t gs = h->bc_stream;
    cudaGraphExec_t execs[3] = {nullptr, nullptr, nullptr};   // sigma, delta, height
    struct ExecGuard {
        cudaGraphExec_t* e;
        ~ExecGuard() {
            for (int j = 0; j < 3; j++)
                if (e[j]) cudaGraphExecDestroy(e[j]);
        }
    } eg{execs};
    // default: graph-captured chunks of R pass launches; PHAST_BC_PERSIST=1 runs every pass
    // of a direction in ONE cooperative launch with a grid barrier between passes
    // (measured slower: the passes are bound by their dependent-load
    // chains, not by launches)
    const char* pe = std::getenv("PHAST_BC_PERSIST");
    const bool persist = pe && pe[0] == '1';
    auto kahn = [&](int which, int backward, auto pass) -> int {
        if (persist) {
            if (cudaMemsetAsync(h->bc_qs, 0, 12, st) != cudaSuccess ||
                launch_bc_count(G, h->dist_scratch, n, k, backward, cnt, qbuf[0], h->bc_qs, st) != cudaSuccess)
                return PHAST_ECUDA;
            void* val = which == 0 ? (void*)h->bc_sigma : (void*)h->bc_delta;
            if (launch_bc_persistent(G, h->dist_scratch, h->bc_sigma, val, k, which, qbuf[0], qbuf[1], h->bc_qs, cnt,
                                     n + 2, h->g.err, st) != cudaSuccess) {
                cudaGetLastError();
                return PHAST_ECUDA;
            }
            return PHAST_OK;
        }
        if (!execs[which]) {
            cudaGraph_t graph = nullptr;
            if (cudaStreamBeginCapture(gs, cudaStreamCaptureModeThreadLocal) != cudaSuccess) return PHAST_ECUDA;
            bool ok = cudaMemsetAsync(h->bc_changed, 0, R * 4, gs) == cudaSuccess;
            for (uint32_t p = 0; ok && p < R; p++) {
                BcQueue Q{qbuf[p % 2], h->bc_qs + p % 3, qbuf[(p + 1) % 2], h->bc_qs + (p + 1) % 3,
                          h->bc_qs + (p + 2) % 3, cnt};
                ok = pass(Q, h->bc_changed + p, gs) == cudaSuccess;
            }
            ok = ok && cudaMemcpyAsync(h->bc_changed_host, h->bc_changed, R * 4, cudaMemcpyDeviceToHost, gs) ==
                           cudaSuccess;
            add_launches(-(int64_t)R);   // captured, not launched
            if (cudaStreamEndCapture(gs, &graph) != cudaSuccess || !ok) {
                cudaGetLastError();
                if (graph) cudaGraphDestroy(graph);
                return PHAST_ECUDA;
            }
            cudaError_t ie = cudaGraphInstantiate(&execs[which], graph, 0);
            cudaGraphDestroy(graph);
            if (ie != cudaSuccess) {
                cudaGetLastError();
                execs[which] = nullptr;
                return PHAST_ECUDA;
            }
        }
        // the count kernel and the chunks run on gs after everything queued on st so far
        if (cudaEventRecord(h->bc_ev, st) != cudaSuccess || cudaStreamWaitEvent(gs, h->bc_ev, 0) != cudaSuccess ||
            cudaMemsetAsync(h->bc_qs, 0, 12, gs) != cudaSuccess ||
            launch_bc_count(G, h->dist_scratch, n, k, backward, cnt, qbuf[0], h->bc_qs, gs) != cudaSuccess)
            return PHAST_ECUDA;
        for (uint64_t it = 0; it <= (uint64_t)n + R; it += R) {
            if (cudaGraphLaunch(execs[which], gs) != cudaSuccess || cudaStreamSynchronize(gs) != cudaSuccess)
                return PHAST_ECUDA;
            add_launches(R);
            for (uint32_t j = 0; j < R; j++)
                if (h->bc_changed_host[j] == 0) return PHAST_OK;   // st waits for nothing: gs is idle
        }
        return PHAST_EINTERNAL;   // cannot happen with lengths > 0
    };
    uint32_t* hgt = reinterpret_cast<uint32_t*>(h->bc_delta);
    for (uint64_t base = 0; base < count; base += k) {
        Sources S;
        const uint32_t kv = (uint32_t)std::min<uint64_t>(k, count - base);
        for (uint32_t i = 0; i < k; i++) S.s[i] = h->L.perm[sources[base + (i < kv ? i : 0)]];
        if ((rc = run_query(h, S, k, h->dist_scratch, nullptr, st))) return rc;
        if (reach) {
            if (cudaMemsetAsync(hgt, 0, elems * 4, st) != cudaSuccess) return PHAST_ECUDA;
            rc = kahn(2, 1, [&](const BcQueue& Q, uint32_t* ch, cudaStream_t s2) {
                return launch_bc_back(G, h->dist_scratch, nullptr, hgt, n, k, 1, Q, ch, s2);
            });
            if (rc) return rc;
            if (launch_reach_accum(h->dist_scratch, hgt, (uint32_t*)out, n, k, kv, st) != cudaSuccess)
                return PHAST_ECUDA;
            continue;
        }
        if (cudaMemsetAsync(h->bc_sigma, 0, elems * 8, st) != cudaSuccess ||
            cudaMemsetAsync(h->bc_delta, 0, elems * 8, st) != cudaSuccess)
            return PHAST_ECUDA;
        rc = kahn(0, 0, [&](const BcQueue& Q, uint32_t* ch, cudaStream_t s2) {
            return launch_bc_sigma(G, h->dist_scratch, h->bc_sigma, n, k, Q, ch, s2);
        });
        if (rc) return rc;
        rc = kahn(1, 1, [&](const BcQueue& Q, uint32_t* ch, cudaStream_t s2) {
            return launch_bc_back(G, h->dist_scratch, h->bc_sigma, h->bc_delta, n, k, 0, Q, ch, s2);
        });
        if (rc) return rc;
        if (launch_bc_accum(h->bc_delta, (double*)out, n, k, kv, S, st) != cudaSuccess) return PHAST_ECUDA;
    }
    return phast_sync(h, stream);
}
}  // namespace

extern "C" {

int phast_betweenness(phast_ctx* h, const uint32_t* sources, uint64_t count, uint32_t k_batch, double* cb_dev,
                      void* stream) {
    return centrality(h, sources, count, k_batch, cb_dev, false, stream);
}

int phast_reach(phast_ctx* h, const uint32_t* sources, uint64_t count, uint32_t k_batch, uint32_t* reach_dev,
                void* stream) {
    return centrality(h, sources, count, k_batch, reach_dev, true, stream);
}

int phast_info(const phast_ctx* h, phast_info_t* o) {
    if (!h || !o) return PHAST_EINVAL;
    std::memset(o, 0, sizeof(*o));
    o->n = h->n;
    o->levels = h->L.levels;
    o->m = h->m;
    o->m_up = h->L.up_arc.size();
    o->m_down = h->L.dn_arc.size();
    uint64_t nt = 0;
    for (uint32_t w : h->tail_bits) nt += (uint64_t)__builtin_popcount(w);
    o->n_tail = nt;
    o->shortcuts = h->shortcuts;
    o->rounds = h->rounds;
    o->device = h->device < 0 ? 0xFFFFFFFFu : (uint32_t)h->device;
    o->layout = h->L.mode;
    o->delta = h->L.delta;
    o->build_seconds = h->build_seconds;
    return PHAST_OK;
}

int phast_level_sizes(const phast_ctx* h, uint32_t* out) {
    if (!h || !out) return PHAST_EINVAL;
    std::memset(out, 0, (size_t)h->L.levels * 4);
    for (uint32_t l : h->L.level) out[l]++;
    return PHAST_OK;
}

int phast_order(const phast_ctx* h, uint32_t* o) {
    if (!h || !o) return PHAST_EINVAL;
    std::memcpy(o, h->L.perm.data(), (size_t)h->n * 4);
    return PHAST_OK;
}

int phast_export(const phast_ctx* h, uint32_t* level, uint32_t* dn_first, uint32_t* dn_tail, uint32_t* dn_len,
                 uint32_t* up_first, uint32_t* up_head, uint32_t* up_len) {
    if (!h) return PHAST_EINVAL;
    const Layout& L = h->L;
    if (level) std::memcpy(level, L.level.data(), L.level.size() * 4);
    if (dn_first) std::memcpy(dn_first, L.dn_first.data(), L.dn_first.size() * 4);
    if (up_first) std::memcpy(up_first, L.up_first.data(), L.up_first.size() * 4);
    for (size_t i = 0; i < L.dn_arc.size(); i++) {
        if (dn_tail) dn_tail[i] = L.dn_arc[i].x;
        if (dn_len) dn_len[i] = L.dn_arc[i].y;
    }
    for (size_t i = 0; i < L.up_arc.size(); i++) {
        if (up_head) up_head[i] = L.up_arc[i].x;
        if (up_len) up_len[i] = L.up_arc[i].y;
    }
    return PHAST_OK;
}

// ---------------------------------------------------------------- save / load
static const char MAGIC[8] = {'P', 'H', 'A', 'S', 'T', 'B', '2', '3'};

int phast_save(const phast_ctx* h, const char* path) {
    if (!h || !path) return PHAST_EINVAL;
    FILE* f = std::fopen(path, "wb");
    if (!f) return PHAST_EIO;
    const Layout& L = h->L;
    uint64_t hdr[10] = {h->n, L.levels, h->m, h->shortcuts, h->rounds, L.dn_arc.size(), L.up_arc.size(),
                        L.mode | ((uint64_t)L.cut << 32) | ((uint64_t)L.lag << 56), L.delta, L.lvl_off.size()};
    auto wr = [&](const void* p, size_t sz, size_t cnt) { return std::fwrite(p, sz, cnt, f) == cnt; };
    bool ok = wr(MAGIC, 1, 8) && wr(hdr, 8, 10) && wr(&h->build_seconds, 8, 1) && wr(L.perm.data(), 4, h->n) &&
              wr(L.level.data(), 4, h->n) && wr(L.lvl_off.data(), 4, L.lvl_off.size()) &&
              wr(L.dn_first.data(), 4, L.dn_first.size()) && wr(L.up_first.data(), 4, L.up_first.size()) &&
              wr(L.dn_arc.data(), 8, L.dn_arc.size()) && wr(L.up_arc.data(), 8, L.up_arc.size());
    const uint64_t n_in = L.in_arc.size();
    ok = ok && wr(&n_in, 8, 1) && wr(L.in_first.data(), 4, L.in_first.size()) && wr(L.in_arc.data(), 8, n_in);
    ok = (std::fclose(f) == 0) && ok;
    return ok ? PHAST_OK : PHAST_EIO;
}

int phast_load(const char* path, uint32_t flags, phast_ctx** out) {
    if (!path || !out) return PHAST_EINVAL;
    *out = nullptr;
    FILE* f = std::fopen(path, "rb");
    if (!f) return PHAST_EIO;
    std::unique_ptr<phast_ctx> h(new (std::nothrow) phast_ctx());
    char magic[8];
    uint64_t hdr[10];
    auto rd = [&](void* p, size_t sz, size_t cnt) { return std::fread(p, sz, cnt, f) == cnt; };
    bool ok = h && rd(magic, 1, 8) && std::memcmp(magic, MAGIC, 8) == 0 && rd(hdr, 8, 10) &&
              rd(&h->build_seconds, 8, 1) && hdr[0] > 0 && hdr[0] < 0xFFFFFFFFull;
    if (ok) {
        Layout& L = h->L;
        try {
            h->n = (uint32_t)hdr[0]; L.levels = (uint32_t)hdr[1]; h->m = hdr[2];
            h->shortcuts = hdr[3]; h->rounds = (uint32_t)hdr[4];
            L.mode = (uint32_t)hdr[7]; L.cut = (uint32_t)((hdr[7] >> 32) & 0xFFFFFFu);
            L.lag = std::max(1u, (uint32_t)(hdr[7] >> 56)); L.delta = (uint32_t)hdr[8];
            L.perm.resize(h->n); L.iperm.resize(h->n); L.level.resize(h->n);
            L.lvl_off.resize(hdr[9]);
            L.dn_first.resize((size_t)h->n + 1); L.up_first.resize((size_t)h->n + 1);
            L.dn_arc.resize(hdr[5]); L.up_arc.resize(hdr[6]);
        } catch (const std::bad_alloc&) {
            std::fclose(f);
            return PHAST_ENOMEM;
        }
        ok = rd(L.perm.data(), 4, h->n) && rd(L.level.data(), 4, h->n) && rd(L.lvl_off.data(), 4, L.lvl_off.size()) &&
             rd(L.dn_first.data(), 4, L.dn_first.size()) && rd(L.up_first.data(), 4, L.up_first.size()) &&
             rd(L.dn_arc.data(), 8, L.dn_arc.size()) && rd(L.up_arc.data(), 8, L.up_arc.size());
        uint64_t n_in = 0;
        ok = ok && rd(&n_in, 8, 1) && n_in < 0xFFFFFFFEull;
        if (ok) {
            try {
                L.in_first.resize((size_t)h->n + 1);
                L.in_arc.resize(n_in);
            } catch (const std::bad_alloc&) {
                std::fclose(f);
                return PHAST_ENOMEM;
            }
            ok = rd(L.in_first.data(), 4, L.in_first.size()) && rd(L.in_arc.data(), 8, n_in) &&
                 L.in_first[h->n] == n_in;
        }
    }
    std::fclose(f);
    if (!ok) return PHAST_EIO;
    for (uint32_t v = 0; v < h->n; v++) {
        if (h->L.perm[v] >= h->n) return PHAST_EIO;
        h->L.iperm[h->L.perm[v]] = v;
    }
    compute_tail_bits(h.get());
    if (!(flags & PHAST_FLAG_HOST_ONLY)) {
        int rc = upload(h.get());
        if (rc) return rc;
    }
    *out = h.release();
    return PHAST_OK;
}

void phast_free(phast_ctx* h) {
    if (!h) return;
    free_device(h);
    delete h;
}

const char* phast_strerror(int s) {
    switch (s) {
        case PHAST_OK: return "ok";
        case PHAST_EINVAL: return "invalid argument";
        case PHAST_ENOMEM: return "out of memory";
        case PHAST_ECUDA: return "CUDA error";
        case PHAST_ERANGE: return "value out of range";
        case PHAST_ESTATE: return "handle has no device image";
        case PHAST_EIO: return "I/O error";
        case PHAST_EINTERNAL: return "internal invariant failed";
        default: return "unknown status";
    }
}

int phast_timing(phast_ctx* h, int enable) {
    if (!h) return PHAST_EINVAL;
    if (h->device < 0) return PHAST_ESTATE;
    if (enable) h->ev_used = 0;
    h->timing = enable != 0;
    return PHAST_OK;
}

int phast_timing_read(phast_ctx* h, double* ms_up, double* ms_sweep, uint64_t* batches) {
    if (!h || !ms_up || !ms_sweep || !batches) return PHAST_EINVAL;
    if (h->device < 0) return PHAST_ESTATE;
    DeviceGuard dg(h->device);
    double a = 0, b = 0;
    for (size_t i = 0; i + 2 < h->ev_used; i += 3) {
        float x = 0, y = 0;
        if (cudaEventSynchronize(h->ev[i + 2]) != cudaSuccess) { cudaGetLastError(); return PHAST_ECUDA; }
        if (cudaEventElapsedTime(&x, h->ev[i], h->ev[i + 1]) != cudaSuccess ||
            cudaEventElapsedTime(&y, h->ev[i + 1], h->ev[i + 2]) != cudaSuccess) {
            cudaGetLastError();
            return PHAST_ECUDA;
        }
        a += x;
        b += y;
    }
    *ms_up = a;
    *ms_sweep = b;
    *batches = h->ev_used / 3;
    return PHAST_OK;
}

int phast_plan_stats(const phast_ctx* h, uint32_t k, uint32_t grid, uint64_t* out) {
    if (!h || !out || !k_ok(k) || grid == 0) return PHAST_EINVAL;
    ChunkPlan cp;
    int rc = plan_chunks(h->L, chunk_cap_for(h->L, k, grid), grid, cp);
    if (rc) return rc;
    out[0] = cp.chunks;
    out[1] = cp.slots;
    out[2] = cp.pads;
    out[3] = (cp.slots + grid - 1) / grid;
    out[4] = chunk_cap_for(h->L, k, grid);
    return PHAST_OK;
}

uint64_t phast_launch_count(void) { return launches(); }

}  // extern "C"
