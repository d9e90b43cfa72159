// capi.cu -- the C ABI of include/phast.h: handle lifetime, validation, device
// image upload, launch plans and query orchestration.
//
// Layout (layout.cpp): internal ids follow a reverse topological order
// of G-down, so that the sweep is "a simple linear sweep in increasing order of IDs"
// (§IV-A).  G-down: in-arcs by head, {tail, len} (§IV-A),
// sentinel dn_first[n].  G-up: out-arcs by tail, {head, len}.
#include <algorithm>
#include <array>
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

static_assert(PHAST_SLOTS == SLOTS, "phast.h and kernels.h disagree on the slot count");

struct phast_ctx {
    uint32_t n = 0;
    uint64_t m = 0, shortcuts = 0, n_tail = 0;
    uint32_t rounds = 0;
    double build_seconds = 0;
    Layout L;
    std::vector<uint8_t> wide;          // per level (top-down): the two-record ELL format (DevImage::dn_rec2)
    phast_query_opts q = {0, 0, 0, 0, 0, 0, 0};
    // upward-search-space statistics of phast_info (host sample, computed once)
    mutable bool up_stats = false;
    mutable double up_mean = 0;
    mutable uint32_t up_max = 0, up_samples = 0;
    // device
    int device = -1;
    DevImage g;
    // per-query slots (PHAST_SLOTS in flight): visited bits + search spaces; upward
    // searches run on their slot's side stream, each waiting for its slot's previous query
    Slot slot[SLOTS];
    cudaEvent_t up_done[SLOTS] = {};
    cudaEvent_t slot_free[SLOTS] = {};
    uint32_t slot_next = 0;
    cudaStream_t side[SLOTS] = {};     // upward searches, one stream per slot (they overlap)
    uint32_t* pad[SLOTS] = {};          // padded-k label scratch per slot (phast_trees with k not a power of two)
    size_t pad_elems[SLOTS] = {};
    // library streams for batches in flight (phast_diameter) and their label buffers
    cudaStream_t lane[SLOTS] = {};
    cudaEvent_t lane_ev[SLOTS] = {};
    cudaEvent_t fork_ev = nullptr;
    uint32_t* lane_dist[SLOTS] = {};
    size_t lane_elems[SLOTS] = {};
    uint32_t* host_scratch = nullptr;   // phast_trees_host label buffer
    size_t host_elems = 0;
    uint32_t* batch_max_scratch = nullptr;
    size_t batch_max_elems = 0;
    uint32_t* wit = nullptr;            // [4] witness scratch: max, pad, 64-bit key
    uint32_t* d_in_first = nullptr;     // original in-CSR on the device (parents; uploaded on first use)
    uint2* d_in_arc = nullptr;
    // NEXT-3 betweenness: original out-CSR {head, len} by tail (internal ids), sigma/delta
    // rows [n][k] fp64, per-pass change words (device + pinned host), label rows
    uint32_t* d_out_first = nullptr;
    uint2* d_out_arc = nullptr;
    double* bc_sigma = nullptr;
    double* bc_delta = nullptr;
    uint32_t* bc_dist = nullptr;
    uint32_t* bc_src = nullptr;         // [B*k] internal ids of a group's trees
    size_t bc_elems = 0;
    uint32_t* bc_changed = nullptr;
    uint32_t* bc_changed_host = nullptr;
    uint32_t* bc_q = nullptr;           // [3][n*k]: two item queues + unfinished-input counts
    uint32_t* bc_qs = nullptr;          // [3] rotating queue sizes
    cudaStream_t bc_stream = nullptr;   // private stream the pass graphs run on
    cudaEvent_t bc_ev = nullptr;
    int bc_len_ok = 0;                  // 0 unknown, 1 all original lengths > 0, -1 not
    // top levels [0, J) swept in one single-CTA launch (launch_sweep_top), one plan per k
    struct Top {
        uint4* chunks = nullptr;   // device [nchunks] {vbeg, vend, first[vbeg], first[vend]}
        uint4* rnd = nullptr;      // device [2 nchunks] rounds of multi-level chunks
        TopArgs a;                 // a.fused: the whole query in this one launch
        uint32_t J = 0;            // levels [0, J) in the shared-memory launch (0: none)
        uint32_t vtop = 0;         // upward searches stop expanding below this id (0: full searches)
        uint32_t* up_f = nullptr;  // top mode with vtop: A-up in-arcs by head inside [0, V)
        uint2* up_a = nullptr;
    };
    std::map<uint32_t, Top> tops;
    // band launches (layout.h Band) per k: work units of consecutive closed groups
    struct BandRun {
        uint32_t* off = nullptr;   // device [F][U+1]
        BandArgs a;
        uint32_t seg_lo = 0, seg_hi = 0;
    };
    std::map<uint32_t, std::vector<BandRun>> bandruns;
    // A-up in-arcs by head {tail, len}, all of them (hierarchy parents; uploaded on first use)
    uint32_t* d_upall_first = nullptr;
    uint2* d_upall_arc = nullptr;
    // A-up in-arcs by head {tail, len} (fused single-launch queries on small graphs)
    uint32_t* d_upin_first = nullptr;
    uint2* d_upin_arc = nullptr;
    bool upin_tried = false;
    // stage timing (phast_timing)
    bool timing = false;
    std::vector<cudaEvent_t> ev;   // 3 per recorded batch
    size_t ev_used = 0;
};

namespace {

constexpr uint32_t SEED_CAP = 1u << 16;   // default per-source search-space capacity
constexpr uint32_t UP_SAMPLE = 1024;      // sources sampled for phast_info's search-space stats
// a level gets the two-record ELL format when more than this share of its vertices have
// more than two in-arcs (C3: levels 2-11 and 14-; 35-81 % of their vertices)
constexpr double WIDE_SHARE = 0.15;

// the vector widths the kernels are instantiated for; any other k runs at the next one
uint32_t kpad(uint32_t k) {
    uint32_t p = 1;
    while (p < k) p *= 2;
    return p;
}
bool k_valid(uint32_t k) { return k >= 1 && k <= KMAX; }

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

// device buffer that only grows
template <class T>
int grow(T** p, size_t* have, size_t elems) {
    if (*have >= elems && *p) return PHAST_OK;
    cudaFree(*p);
    *p = nullptr;
    *have = 0;
    int rc = dmalloc(p, elems);
    if (!rc) *have = elems;
    return rc;
}

void free_tops(phast_ctx* h) {
    for (auto& kv : h->tops) {
        cudaFree(kv.second.chunks);
        cudaFree(kv.second.rnd);
        cudaFree(kv.second.up_f);
        cudaFree(kv.second.up_a);
    }
    h->tops.clear();
    for (auto& kv : h->bandruns)
        for (auto& b : kv.second) cudaFree(b.off);
    h->bandruns.clear();
}

void free_seeds(phast_ctx* h) {
    for (uint32_t s = 0; s < SLOTS; s++) {
        cudaFree(h->slot[s].seed_v);
        cudaFree(h->slot[s].seed_d);
        h->slot[s].seed_v = h->slot[s].seed_d = nullptr;
    }
    for (uint32_t s = 0; s < SLOTS; s++) {
        cudaFree(h->slot[s].gscratch);
        h->slot[s].gscratch = nullptr;
    }
}

// search-space buffers for the current options (phast_query_opts seed_cap / up_smem_cap)
int alloc_seeds(phast_ctx* h) {
    auto pow2 = [](uint32_t x) { uint32_t p = 1; while (p * 2 <= x) p *= 2; return p; };
    const uint32_t cap = h->q.seed_cap ? std::max(16u, std::min(SEED_CAP, h->q.seed_cap)) : SEED_CAP;
    const uint32_t sm = h->q.up_smem_cap ? std::max(16u, std::min(4096u, h->q.up_smem_cap)) : 4096u;
    h->g.seed_cap = pow2(cap);
    // a shared-memory table never holds more than the per-source capacity (a search
    // that outgrows it continues in the global table, which reports the overflow)
    h->g.smem_cap = std::min(pow2(sm), h->g.seed_cap);
    int rc;
    for (uint32_t s = 0; s < SLOTS; s++)
        if ((rc = dmalloc(&h->slot[s].seed_v, (size_t)KMAX * h->g.seed_cap)) ||
            (rc = dmalloc(&h->slot[s].seed_d, (size_t)KMAX * h->g.seed_cap)))
            return rc;
    for (uint32_t s = 0; s < SLOTS; s++)
        if ((rc = dmalloc(&h->slot[s].gscratch, (size_t)KMAX * h->g.seed_cap * 5))) return rc;
    return PHAST_OK;
}

void free_device(phast_ctx* h) {
    if (h->device < 0) return;
    DeviceGuard dg(h->device);
    cudaDeviceSynchronize();
    free_tops(h);
    free_seeds(h);
    for (cudaEvent_t e : h->ev) cudaEventDestroy(e);
    h->ev.clear();
    h->ev_used = 0;
    for (uint32_t s = 0; s < SLOTS; s++) {
        if (h->up_done[s]) cudaEventDestroy(h->up_done[s]);
        if (h->slot_free[s]) cudaEventDestroy(h->slot_free[s]);
        if (h->lane_ev[s]) cudaEventDestroy(h->lane_ev[s]);
        if (h->lane[s]) cudaStreamDestroy(h->lane[s]);
        cudaFree(h->slot[s].flags);
        cudaFree(h->slot[s].seed_cnt);
        cudaFree(h->pad[s]);
        cudaFree(h->lane_dist[s]);
        h->up_done[s] = h->slot_free[s] = h->lane_ev[s] = nullptr;
        h->lane[s] = nullptr;
        h->slot[s] = Slot();
        h->pad[s] = h->lane_dist[s] = nullptr;
        h->pad_elems[s] = h->lane_elems[s] = 0;
    }
    if (h->fork_ev) cudaEventDestroy(h->fork_ev);
    h->fork_ev = nullptr;
    for (uint32_t s = 0; s < SLOTS; s++) {
        if (h->side[s]) cudaStreamDestroy(h->side[s]);
        h->side[s] = nullptr;
    }
    cudaFree((void*)h->g.dn_first); cudaFree((void*)h->g.dn_arc);
    cudaFree((void*)h->g.dn_rec); cudaFree((void*)h->g.dn_rec2); cudaFree((void*)h->g.dn_ovf);
    cudaFree((void*)h->g.up_first); cudaFree((void*)h->g.up_arc);
    cudaFree(h->g.err);
    cudaFree(h->host_scratch); cudaFree(h->batch_max_scratch); cudaFree(h->wit);
    cudaFree(h->d_in_first); cudaFree(h->d_in_arc);
    cudaFree(h->d_out_first); cudaFree(h->d_out_arc);
    cudaFree(h->bc_sigma); cudaFree(h->bc_delta); cudaFree(h->bc_dist); cudaFree(h->bc_src);
    cudaFree(h->bc_changed); cudaFreeHost(h->bc_changed_host); cudaFree(h->bc_q); cudaFree(h->bc_qs);
    if (h->bc_stream) cudaStreamDestroy(h->bc_stream);
    if (h->bc_ev) cudaEventDestroy(h->bc_ev);
    cudaFree(h->d_upin_first); cudaFree(h->d_upin_arc);
    cudaFree(h->d_upall_first); cudaFree(h->d_upall_arc);
    h->d_upall_first = nullptr; h->d_upall_arc = nullptr;
    h->host_scratch = nullptr; h->host_elems = 0;
    h->batch_max_scratch = nullptr; h->batch_max_elems = 0; h->wit = nullptr;
    h->d_in_first = nullptr; h->d_in_arc = nullptr;
    h->d_out_first = nullptr; h->d_out_arc = nullptr;
    h->bc_sigma = h->bc_delta = nullptr; h->bc_dist = nullptr; h->bc_src = nullptr; h->bc_elems = 0;
    h->bc_changed = nullptr; h->bc_changed_host = nullptr; h->bc_q = nullptr; h->bc_qs = nullptr;
    h->bc_stream = nullptr; h->bc_ev = nullptr;
    h->d_upin_first = nullptr; h->d_upin_arc = nullptr; h->upin_tried = false;
    h->g = DevImage();
    h->device = -1;
}

void count_tails(phast_ctx* h) {
    std::vector<uint32_t> bits(((size_t)h->n + 31) / 32, 0u);
    for (const Arc& a : h->L.dn_arc) bits[a.x >> 5] |= 1u << (a.x & 31);
    uint64_t nt = 0;
    for (uint32_t w : bits) nt += (uint64_t)__builtin_popcount(w);
    h->n_tail = nt;
}

int upload(phast_ctx* h) {
    int dev = 0;
    if (cudaGetDevice(&dev) != cudaSuccess) { cudaGetLastError(); return PHAST_ECUDA; }
    h->device = dev;
    DevImage& g = h->g;
    g.n = h->n;
    const Layout& L = h->L;
    uint32_t *dnf = nullptr, *upf = nullptr;
    uint2 *dna = nullptr, *upa = nullptr;
    int rc;
    const size_t nw = ((size_t)h->n + 31) / 32;
    // +4 / +2 elements: 16-byte aligned bulk copies may read up to 12 bytes past the end
    if ((rc = dmalloc(&dnf, L.dn_first.size() + 4)) || (rc = dmalloc(&dna, L.dn_arc.size() + 2)) ||
        (rc = dmalloc(&upf, L.up_first.size())) || (rc = dmalloc(&upa, L.up_arc.size())) ||
        (rc = dmalloc(&g.err, 1))) {
        g.dn_first = dnf; g.dn_arc = dna; g.up_first = upf; g.up_arc = upa;
        free_device(h);
        return rc;
    }
    g.dn_first = dnf; g.dn_arc = dna; g.up_first = upf; g.up_arc = upa;
    for (uint32_t s = 0; s < SLOTS; s++)
        if ((rc = dmalloc(&h->slot[s].flags, nw + 4)) || (rc = dmalloc(&h->slot[s].seed_cnt, KMAX))) {
            free_device(h);
            return rc;
        }
    if ((rc = alloc_seeds(h))) {
        free_device(h);
        return rc;
    }
    // G-down as ELL records + overflow lists (kernels.h: DevImage::dn_rec / dn_rec2); a
    // level is "wide" when more than WIDE_SHARE of its vertices have more than two in-arcs
    {
        const uint32_t nseg = (uint32_t)L.lvl_off.size() - 1;
        h->wide.assign(nseg, 0);
        bool any_wide = false;
        for (uint32_t j = 0; j < nseg; j++) {
            uint32_t many = 0;
            for (uint32_t v = L.lvl_off[j]; v < L.lvl_off[j + 1]; v++) many += L.dn_first[v + 1] - L.dn_first[v] > 2;
            h->wide[j] = (double)many > WIDE_SHARE * (L.lvl_off[j + 1] - L.lvl_off[j]) ? 1 : 0;
            any_wide |= h->wide[j] != 0;
        }
        std::vector<uint4> rec(h->n), rec2(any_wide ? h->n : 0, make_uint4(INF, INF, INF, INF));
        std::vector<Arc> ovf;
        for (uint32_t j = 0; j < nseg; j++)
            for (uint32_t v = L.lvl_off[j]; v < L.lvl_off[j + 1]; v++) {
                const uint32_t e0 = L.dn_first[v], deg = L.dn_first[v + 1] - e0;
                const Arc* a = L.dn_arc.data() + e0;
                uint4 r = make_uint4(INF, INF, INF, INF);
                if (deg >= 1) { r.x = a[0].x; r.y = a[0].y; }
                if (h->wide[j]) {   // arcs 0-1 | 2-3, or 2 + overflow
                    if (deg >= 2) { r.z = a[1].x; r.w = a[1].y; }
                    uint4 r2 = make_uint4(INF, INF, INF, INF);
                    if (deg >= 3) { r2.x = a[2].x; r2.y = a[2].y; }
                    if (deg == 4) { r2.z = a[3].x; r2.w = a[3].y; }
                    if (deg > 4) {
                        r2.z = (uint32_t)ovf.size();
                        ovf.push_back(Arc{deg - 3, 0});
                        for (uint32_t e = 3; e < deg; e++) ovf.push_back(a[e]);
                    }
                    rec2[v] = r2;
                } else {            // arcs 0-1, or 0 + overflow
                    if (deg == 2) { r.z = a[1].x; r.w = a[1].y; }
                    if (deg > 2) {
                        r.z = (uint32_t)ovf.size();
                        ovf.push_back(Arc{deg - 1, 0});
                        for (uint32_t e = 1; e < deg; e++) ovf.push_back(a[e]);
                    }
                }
                rec[v] = r;
            }
        uint4 *dr = nullptr, *dr2 = nullptr;
        uint2* dov = nullptr;
        if (ovf.size() >= INF || (rc = dmalloc(&dr, rec.size())) || (rc = dmalloc(&dov, ovf.size())) ||
            (any_wide && (rc = dmalloc(&dr2, rec2.size())))) {
            cudaFree(dr);
            cudaFree(dov);
            free_device(h);
            return rc ? rc : PHAST_ERANGE;
        }
        g.dn_rec = dr;
        g.dn_rec2 = dr2;
        g.dn_ovf = dov;
        if (cudaMemcpy(dr, rec.data(), rec.size() * sizeof(uint4), cudaMemcpyHostToDevice) != cudaSuccess ||
            (any_wide && cudaMemcpy(dr2, rec2.data(), rec2.size() * sizeof(uint4), cudaMemcpyHostToDevice) != cudaSuccess) ||
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
              cudaMemset(g.err, 0, 4) == cudaSuccess &&

              cudaEventCreateWithFlags(&h->fork_ev, cudaEventDisableTiming) == cudaSuccess;
    for (uint32_t s = 0; ok && s < SLOTS; s++)
        ok = cudaMemset(h->slot[s].flags, 0, (nw + 4) * 4) == cudaSuccess &&
             cudaMemset(h->slot[s].seed_cnt, 0, KMAX * 4) == cudaSuccess &&
             cudaEventCreateWithFlags(&h->up_done[s], cudaEventDisableTiming) == cudaSuccess &&
             cudaEventCreateWithFlags(&h->slot_free[s], cudaEventDisableTiming) == cudaSuccess &&
             cudaEventCreateWithFlags(&h->lane_ev[s], cudaEventDisableTiming) == cudaSuccess &&
             cudaStreamCreateWithFlags(&h->lane[s], cudaStreamNonBlocking) == cudaSuccess &&
             cudaStreamCreateWithFlags(&h->side[s], cudaStreamNonBlocking) == cudaSuccess;
    ok = ok && cudaDeviceSynchronize() == cudaSuccess;
    if (!ok) { cudaGetLastError(); free_device(h); return PHAST_ECUDA; }
    return PHAST_OK;
}

int validate_csr(uint32_t n, const uint64_t* first, const uint32_t* head, const uint32_t* len) {
    if (n == 0 || n == 0xFFFFFFFFu || !first) return PHAST_EINVAL;
    if (first[0] != 0) return PHAST_EINVAL;
    for (uint32_t v = 0; v < n; v++)
        if (first[v + 1] < first[v]) return PHAST_EINVAL;
    const uint64_t m = first[n];
    if (m && (!head || !len)) return PHAST_EINVAL;
    for (uint64_t e = 0; e < m; e++)
        if (head[e] >= n) return PHAST_EINVAL;
    return PHAST_OK;
}

// a0: original ids -> internal ids; the kp - k padding trees repeat sources[0]
int map_sources(const phast_ctx* h, const uint32_t* src, uint32_t k, uint32_t kp, Sources& S) {
    for (uint32_t i = 0; i < k; i++) {
        if (src[i] >= h->n) return PHAST_ERANGE;
        S.s[i] = h->L.perm[src[i]];
    }
    for (uint32_t i = k; i < KMAX; i++) S.s[i] = i < kp ? S.s[0] : 0u;
    return PHAST_OK;
}

// Multi-level chunks: runs of adjacent chunks [from, ch.size()) (one direction of the
// top plan, in processing order) whose items together fit one warp -- (vertices) x G
// <= 32, no heavy vertex, arcs within the stage -- become one chunk of consecutive ids
// with a round per item (top.cu): round(v) = 1 + the largest round of v's tails inside
// the chunk, 0 if none.  `up`: the chunks run in ascending levels (descending ids;
// tails have larger ids), else descending levels (tails have smaller ids).
void merge_tiny(std::vector<uint4>& ch, size_t from, const uint32_t* f, const std::vector<Arc>& arc, uint32_t G,
                bool big, bool up, std::vector<std::array<uint8_t, 32>>& rnd, bool enabled) {
    if (!enabled) return;
    const uint32_t ECH = top_chunk_arcs(big), VM = top_chunk_vertices(big), HB = 0x80000000u;
    std::vector<uint4> out(ch.begin(), ch.begin() + from);
    std::vector<std::array<uint8_t, 32>> rout(rnd.begin(), rnd.begin() + from);
    size_t i = from;
    auto lanes = [&](const uint4& c) { return (uint64_t)((c.y & 0x3FFFFFFFu) - c.x) * G; };
    while (i < ch.size()) {
        size_t j = i + 1;
        uint32_t vb = ch[i].x, ve = ch[i].y & 0x3FFFFFFFu;
        if (!(ch[i].y & HB) && lanes(ch[i]) <= 32) {
            while (j < ch.size() && !(ch[j].y & HB)) {
                const uint32_t jb = ch[j].x, je = ch[j].y & 0x3FFFFFFFu;
                const bool adj = up ? je == vb : jb == ve;
                const uint32_t nb = up ? jb : vb, ne = up ? ve : je;
                if (!adj || (uint64_t)(ne - nb) * G > 32 || ne - nb > VM || f[ne] - f[nb] > ECH) break;
                vb = nb;
                ve = ne;
                j++;
            }
        }
        if (j == i + 1) {   // nothing to merge
            out.push_back(ch[i]);
            rout.push_back({});
            i++;
            continue;
        }
        std::array<uint8_t, 32> r{};
        std::vector<uint32_t> rv(ve - vb, 0);
        for (uint32_t s = 0; s < ve - vb; s++) {
            const uint32_t v = up ? ve - 1 - s : vb + s;   // tails first
            uint32_t m = 0;
            for (uint32_t e = f[v]; e < f[v + 1]; e++)
                if (arc[e].x >= vb && arc[e].x < ve) m = std::max(m, rv[arc[e].x - vb] + 1);
            rv[v - vb] = std::min(m, 255u);
        }
        for (uint32_t x = 0; x < (ve - vb) * G; x++) r[x] = (uint8_t)rv[x / G];
        out.push_back(make_uint4(vb, ve | top_multi_bit(), f[vb], f[ve]));
        rout.push_back(r);
        i = j;
    }
    ch.swap(out);
    rnd.swap(rout);
}

// Chunks of one level [a, b) over a CSR (offsets `f`): <= VCH vertices and <= ECH
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

// A-up in-arcs by head {tail, len} of the arcs inside [0, V) (V = n: all of them; the
// top levels are a prefix of the ids and A-up climbs, so a tail < V has its head < V),
// as a CSR over [0, V]; false if some head has more than `cap` in-arcs.  Arcs entering
// [0, V) from below are the upward search's (hybrid mode): the pull pass reads only
// rows inside [0, V), which live in shared memory.
bool upin_csr(const Layout& L, uint32_t V, uint32_t cap, std::vector<uint32_t>& f, std::vector<Arc>& arc) {
    f.assign((size_t)V + 1, 0);
    for (uint32_t u = 0; u < V; u++)
        for (uint32_t e = L.up_first[u]; e < L.up_first[u + 1]; e++) f[L.up_arc[e].x + 1]++;
    for (uint32_t v = 0; v < V; v++) {
        if (f[v + 1] > cap) return false;
        f[v + 1] += f[v];
    }
    arc.resize(f[V]);
    std::vector<uint32_t> pos(f.begin(), f.end() - 1);
    for (uint32_t u = 0; u < V; u++)
        for (uint32_t e = L.up_first[u]; e < L.up_first[u + 1]; e++) arc[pos[L.up_arc[e].x]++] = Arc{u, L.up_arc[e].y};
    return true;
}

// upload a CSR with the bulk-copy padding (+4 offsets, +2 arcs)
bool upload_csr(const std::vector<uint32_t>& f, const std::vector<Arc>& arc, uint32_t** df, uint2** da) {
    *df = nullptr;
    *da = nullptr;
    if (dmalloc(df, f.size() + 4) || dmalloc(da, arc.size() + 2)) {
        cudaFree(*df);
        *df = nullptr;
        return false;
    }
    if (cudaMemset(*df, 0, (f.size() + 4) * 4) != cudaSuccess || cudaMemset(*da, 0, (arc.size() + 2) * 8) != cudaSuccess ||
        cudaMemcpy(*df, f.data(), f.size() * 4, cudaMemcpyHostToDevice) != cudaSuccess ||
        (!arc.empty() && cudaMemcpy(*da, arc.data(), arc.size() * 8, cudaMemcpyHostToDevice) != cudaSuccess)) {
        cudaGetLastError();
        cudaFree(*df);
        cudaFree(*da);
        *df = nullptr;
        *da = nullptr;
        return false;
    }
    return true;
}

// Shared-memory sweep plan (top.cu: sweep_top_kernel) for one k; nullptr = none (every
// level gets its own launch):
//  - fused: the whole graph's rows fit the label budget -> the whole query (G-up pull
//    sweep, then the G-down sweep) in one launch (off with PHAST_Q_NO_FUSED);
//  - top: the longest prefix of levels whose rows [0, V) fit, each level small enough
//    for one SM (<= 32 items per consumer thread); the rest one launch per level (off
//    with PHAST_Q_NO_TOP; V capped by top_max_vertices).
// Both need every vertex to have at most top_chunk_arcs(big) in-arcs; big chunks
// (top_big_fits) when the rows leave room for them.
phast_ctx::Top* get_top(phast_ctx* h, uint32_t k) {
    auto it = h->tops.find(k);
    if (it != h->tops.end()) return it->second.chunks ? &it->second : nullptr;
    phast_ctx::Top& T = h->tops[k];   // chunks stays nullptr: "no plan"
    const Layout& L = h->L;
    if (L.lvl_off.size() < 2 || h->n >= 0x40000000u) return nullptr;   // chunk vend carries two flag bits
    const uint32_t nseg = (uint32_t)L.lvl_off.size() - 1;
    const uint32_t G = k >= 4 ? k / 4 : 1;
    const uint64_t vmax_budget = top_label_budget() / (4ull * k);
    std::vector<uint4> ch;
    bool fused = !(h->q.flags & PHAST_Q_NO_FUSED) && h->n <= vmax_budget;
    const bool fbig = fused && top_big_fits(k, h->n);
    for (uint32_t v = 0; fused && v < h->n; v++) fused = L.dn_first[v + 1] - L.dn_first[v] <= top_chunk_arcs(fbig);
    if (fused && !h->upin_tried) {   // A-up in-arcs by head, uploaded once
        h->upin_tried = true;
        std::vector<uint32_t> f;
        std::vector<Arc> arc;
        if (upin_csr(L, h->n, top_chunk_arcs(true), f, arc)) upload_csr(f, arc, &h->d_upin_first, &h->d_upin_arc);
    }
    std::vector<uint32_t> uf;
    if (fused && h->d_upin_first) {
        uf.resize((size_t)h->n + 1);
        if (cudaMemcpy(uf.data(), h->d_upin_first, uf.size() * 4, cudaMemcpyDeviceToHost) != cudaSuccess) {
            cudaGetLastError();
            return nullptr;
        }
        for (uint32_t v = 0; fused && v < h->n; v++) fused = uf[v + 1] - uf[v] <= top_chunk_arcs(fbig);
    } else {
        fused = false;
    }
    std::vector<std::array<uint8_t, 32>> rnd;
    if (fused) {
        std::vector<uint32_t> hf;
        std::vector<Arc> ha;
        upin_csr(L, h->n, top_chunk_arcs(true), hf, ha);
        for (uint32_t j = nseg; j-- > 0;) push_chunks(ch, uf.data(), L.lvl_off[j], L.lvl_off[j + 1], fbig);   // ascending
        rnd.resize(ch.size());
        merge_tiny(ch, 0, hf.data(), ha, G, fbig, true, rnd, !(h->q.flags & PHAST_Q_NO_MULTI));
        T.a.split = (uint32_t)ch.size();
        const size_t d0 = ch.size();
        for (uint32_t j = 0; j < nseg; j++) push_chunks(ch, L.dn_first.data(), L.lvl_off[j], L.lvl_off[j + 1], fbig);
        rnd.resize(ch.size());
        merge_tiny(ch, d0, L.dn_first.data(), L.dn_arc, G, fbig, false, rnd, !(h->q.flags & PHAST_Q_NO_MULTI));
        T.a.big = fbig;
        T.a.first[0] = h->d_upin_first;
        T.a.arcs[0] = h->d_upin_arc;
        T.a.fused = 1;
        T.J = nseg;
        T.a.V = h->n;
    } else {
        if (h->q.flags & PHAST_Q_NO_TOP) return nullptr;
        uint64_t vmax = vmax_budget;
        if (h->q.top_max_vertices) vmax = std::min<uint64_t>(vmax, h->q.top_max_vertices);
        uint32_t J = 0;
        while (J < nseg) {
            const uint32_t a = L.lvl_off[J], b = L.lvl_off[J + 1];
            if (b > vmax || (uint64_t)(b - a) * G > 32ull * 992) break;
            bool fits = true;
            for (uint32_t v = a; v < b && fits; v++) fits = L.dn_first[v + 1] - L.dn_first[v] <= top_chunk_arcs(false);
            if (!fits) break;
            J++;
        }
        if (J < 2) return nullptr;
        // hybrid upward search: the upward kernel expands only vertices below the top
        // levels; the top kernel finishes G-up inside [0, V) with a pull pass in
        // ascending level order (reading R9), then sweeps G-down.  Exact: a G-up path
        // only climbs, so it enters [0, V) once and its part below V is found by the
        // search, its part inside by the pull pass.
        // When: the upward searches run beside the previous batch's sweep (side stream),
        // so moving work from them into the top kernel only pays when they are the
        // critical path, i.e. when a sweep is shorter than the searches: estimated sweep
        // 8kn B at ~5 TB/s vs ~2 us per search wave (<= one per level).  Measured (r43):
        // C2 k=16 14.1 vs 14.9 us/tree, C2D 50.9 vs 61.5 (hybrid); C2 k=64 3.87 vs 3.60,
        // C3 k=64 2.069 vs 2.058 ms/step (full searches).
        const uint32_t V = L.lvl_off[J];
        const bool big = top_big_fits(k, V);
        T.a.big = big;
        const double sweep_us = 8.0 * k * h->n / 5e6, search_us = 2.0 * L.levels;
        const bool hybrid = (h->q.flags & PHAST_Q_HYBRID_ON) ? true
                            : (h->q.flags & PHAST_Q_HYBRID_OFF) ? false
                                                                 : sweep_us < search_us;
        if (hybrid) {
            std::vector<uint32_t> f;
            std::vector<Arc> arc;
            if (upin_csr(L, V, top_chunk_arcs(big), f, arc) && upload_csr(f, arc, &T.up_f, &T.up_a)) {
                for (uint32_t j = J; j-- > 0;) push_chunks(ch, f.data(), L.lvl_off[j], L.lvl_off[j + 1], big);
                rnd.resize(ch.size());
                merge_tiny(ch, 0, f.data(), arc, G, big, true, rnd, !(h->q.flags & PHAST_Q_NO_MULTI));
                T.a.first[0] = T.up_f;
                T.a.arcs[0] = T.up_a;
                T.vtop = V;
            }
        }
        T.a.split = (uint32_t)ch.size();
        const size_t d0 = ch.size();
        for (uint32_t j = 0; j < J; j++) push_chunks(ch, L.dn_first.data(), L.lvl_off[j], L.lvl_off[j + 1], big);
        rnd.resize(ch.size());
        merge_tiny(ch, d0, L.dn_first.data(), L.dn_arc, G, big, false, rnd, !(h->q.flags & PHAST_Q_NO_MULTI));
        T.J = J;
        T.a.V = V;
    }
    const bool none = ch.empty();
    if (none) ch.push_back(make_uint4(0, 0, 0, 0));   // keep a valid device array
    rnd.resize(ch.size());
    uint4* dch = nullptr;
    uint4* drn = nullptr;
    if (dmalloc(&dch, ch.size()) || dmalloc(&drn, 2 * ch.size()) ||
        cudaMemcpy(dch, ch.data(), ch.size() * sizeof(uint4), cudaMemcpyHostToDevice) != cudaSuccess ||
        cudaMemcpy(drn, rnd.data(), rnd.size() * 32, cudaMemcpyHostToDevice) != cudaSuccess) {
        cudaGetLastError();
        cudaFree(dch);
        cudaFree(drn);
        return nullptr;
    }
    T.chunks = dch;
    T.rnd = drn;
    T.a.chunks = dch;
    T.a.rnd = drn;
    T.a.nchunks = none ? 0u : (uint32_t)ch.size();
    T.a.first[1] = h->g.dn_first;
    T.a.arcs[1] = h->g.dn_arc;
    return &T;
}

// Band launches for k (layout.h Band, sweep.cu band_kernel): each band's closed groups
// merged into work units of at least `target` vertices (phast_query_opts band_unit,
// default 8192 / k: 32 KB of rows per unit), fewer when the band has too few vertices
// to give every resident CTA two units.
int get_bands(phast_ctx* h, uint32_t k, std::vector<phast_ctx::BandRun>** out) {
    *out = nullptr;
    auto it = h->bandruns.find(k);
    if (it != h->bandruns.end()) { *out = &it->second; return PHAST_OK; }
    std::vector<phast_ctx::BandRun> runs;
    // defaults measured on C3: 256-thread CTAs, variant 13 for k >= 32
    // (records one item ahead, tail rows through the L1, two 16-byte lanes per thread),
    // 5 for k = 16 (one lane per thread: equal at C3, 3 % faster at C2), units of 32768 / k
    // vertices (128 KB of rows)
    const uint32_t threads = h->q.band_threads ? h->q.band_threads : 256u;
    const uint32_t variant = k < 16 ? 0u : h->q.band_variant ? h->q.band_variant : k >= 32 ? 13u : 5u;
    const uint64_t resident = (uint64_t)num_sms() * band_sm_threads(variant, threads) / threads;
    int rc = PHAST_OK;
    for (const Band& B : h->L.bands) {
        const uint32_t F = B.seg_hi - B.seg_lo, NG = B.ngroups;
        const uint64_t total = h->L.lvl_off[B.seg_hi] - h->L.lvl_off[B.seg_lo];
        uint64_t target = h->q.band_unit ? h->q.band_unit : std::max<uint32_t>(BAND_GROUP_MIN, 32768 / k);
        target = std::min<uint64_t>(target, std::max<uint64_t>(BAND_GROUP_MIN, total / (2 * resident)));
        std::vector<uint32_t> ub{0};
        uint64_t acc = 0;
        for (uint32_t g = 0; g < NG; g++) {
            for (uint32_t j = 0; j < F; j++) acc += B.goff[(size_t)j * (NG + 1) + g + 1] - B.goff[(size_t)j * (NG + 1) + g];
            if (acc >= target || g + 1 == NG) { ub.push_back(g + 1); acc = 0; }
        }
        const uint32_t U = (uint32_t)ub.size() - 1;
        std::vector<uint32_t> off((size_t)F * (U + 1));
        for (uint32_t j = 0; j < F; j++)
            for (uint32_t u = 0; u <= U; u++) off[(size_t)j * (U + 1) + u] = B.goff[(size_t)j * (NG + 1) + ub[u]];
        phast_ctx::BandRun r;
        if ((rc = dmalloc(&r.off, off.size()))) break;
        runs.push_back(r);
        if (cudaMemcpy(runs.back().off, off.data(), off.size() * 4, cudaMemcpyHostToDevice) != cudaSuccess) {
            cudaGetLastError();
            rc = PHAST_ECUDA;
            break;
        }
        phast_ctx::BandRun& b = runs.back();
        b.seg_lo = B.seg_lo;
        b.seg_hi = B.seg_hi;
        b.a.off = b.off;
        b.a.F = F;
        b.a.U = U;
        b.a.threads = threads;
        b.a.variant = variant;
        for (uint32_t j = 0; j < F && j < 32; j++) b.a.wide |= (h->wide[B.seg_lo + j] ? 1u : 0u) << j;
    }
    if (rc) {
        for (auto& b : runs) cudaFree(b.off);
        return rc;
    }
    auto& slot = h->bandruns[k];
    slot = std::move(runs);
    *out = &slot;
    return PHAST_OK;
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

struct QueryOut {
    uint32_t* dist;            // rows of the sweep (width kp)
    uint32_t* diam = nullptr;  // fused max (a5); rows of level 0 are then not stored
    uint32_t* compact_to = nullptr;   // copy the first kc columns here (padded k)
    uint32_t kc = 0;
    bool nogather = false;     // probe A34
};

// One full query (a0 done; a1-a3, a5) of kp mapped sources on stream st, in the next slot.
int run_query(phast_ctx* h, const Sources& S, uint32_t kp, const QueryOut& o, cudaStream_t st) {
    cudaEvent_t e0 = nullptr, e1 = nullptr, e2 = nullptr;
    if (h->timing && h->ev_used + 3 <= 3 * MAX_TIMED_BATCHES) {
        e0 = timing_event(h); e1 = timing_event(h); e2 = timing_event(h);
        if (!e0 || !e1 || !e2) return PHAST_ECUDA;
        if (cudaEventRecord(e0, st) != cudaSuccess) return PHAST_ECUDA;
    }
    phast_ctx::Top* top = get_top(h, kp);
    const uint32_t s = h->slot_next;
    h->slot_next = (h->slot_next + 1) % SLOTS;
    const Slot& sl = h->slot[s];
    if (top && top->a.fused && !o.nogather) {   // small graph: the whole query (a1-a3, a5) in one launch
        if (e1) cudaEventRecord(e1, st);          // no separate upward stage: all of it is the sweep
        if (launch_sweep_top(top->a, kp, S, o.dist, sl.flags, o.diam, st) != cudaSuccess) return PHAST_ECUDA;
        if (o.compact_to && launch_compact(o.dist, kp, o.compact_to, o.kc, h->n, st) != cudaSuccess)
            return PHAST_ECUDA;
        if (cudaEventRecord(h->slot_free[s], st) != cudaSuccess) return PHAST_ECUDA;   // padded scratch reusable
        if (e2) cudaEventRecord(e2, st);
        return PHAST_OK;
    }
    if (top && top->a.fused) top = nullptr;   // the A34 probe runs every level as its own launch
    // a1 on the slot's side stream (overlaps earlier sweeps and the other slots' searches), after this slot's previous query
    if (cudaStreamWaitEvent(h->side[s], h->slot_free[s], 0) != cudaSuccess) return PHAST_ECUDA;
    if (launch_upward(h->g, sl, S, kp, top ? top->vtop : 0u, h->side[s]) != cudaSuccess) return PHAST_ECUDA;
    if (cudaEventRecord(h->up_done[s], h->side[s]) != cudaSuccess) return PHAST_ECUDA;
    if (cudaStreamWaitEvent(st, h->up_done[s], 0) != cudaSuccess) return PHAST_ECUDA;
    // a2 on the caller's stream
    if (launch_seed(h->g, sl, kp, o.dist, st) != cudaSuccess) return PHAST_ECUDA;
    if (e1) cudaEventRecord(e1, st);
    // a3 + a4: the small top levels in one single-CTA launch, then one launch per level
    // (§VI "The CPU starts, for each level i, a kernel on the GPU")
    const uint32_t levels = (uint32_t)h->L.lvl_off.size() - 1;
    uint32_t j0 = 0;
    if (top) {
        if (launch_sweep_top(top->a, kp, S, o.dist, sl.flags, o.diam, st) != cudaSuccess) return PHAST_ECUDA;
        j0 = top->J;
    }
    // then every band below the top launch in one launch each (a band that reaches into
    // the top launch's levels is swept per level), every other level in its own launch
    std::vector<phast_ctx::BandRun>* bands = nullptr;
    if (!o.nogather && !(h->q.flags & PHAST_Q_NO_BANDS) && !h->L.bands.empty()) {
        const int rc = get_bands(h, kp, &bands);
        if (rc) return rc;
    }
    size_t bi = 0;
    for (uint32_t j = j0; j < levels;) {
        while (bands && bi < bands->size() && (*bands)[bi].seg_lo < j) bi++;
        if (bands && bi < bands->size() && (*bands)[bi].seg_lo == j) {
            const phast_ctx::BandRun& b = (*bands)[bi++];
            BandArgs a = b.a;
            a.store_last = !(o.diam && b.seg_hi == levels);   // level-0 rows are never read again
            a.stream_last = b.seg_hi == levels;
            if (launch_sweep_band(h->g, a, sl.flags, kp, o.dist, o.diam, st) != cudaSuccess) return PHAST_ECUDA;
            j = b.seg_hi;
            continue;
        }
        const bool last = (j + 1 == levels);
        const bool store = !(o.diam && last);   // level-0 rows are never read again (diameter mode)
        if (launch_sweep_level(h->g, sl.flags, kp, h->L.lvl_off[j], h->L.lvl_off[j + 1], o.dist, o.diam, store, last,
                               o.nogather, h->wide[j] != 0, st) != cudaSuccess)
            return PHAST_ECUDA;
        j++;
    }
    if (launch_clear_flags(sl, kp, h->g.seed_cap, st) != cudaSuccess) return PHAST_ECUDA;
    if (o.compact_to && launch_compact(o.dist, kp, o.compact_to, o.kc, h->n, st) != cudaSuccess) return PHAST_ECUDA;
    // the slot (visited bits, search space, padded scratch) is free for the query SLOTS later
    if (cudaEventRecord(h->slot_free[s], st) != cudaSuccess) return PHAST_ECUDA;
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
    if (h->d_in_first) return PHAST_OK;   // the original in-CSR, uploaded on first use (parents, centrality)
    uint32_t* f = nullptr;
    uint2* a = nullptr;
    int rc;
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
    return PHAST_OK;
}

// Original out-arcs by tail {head, len} in internal ids: the transpose of L.in_arc
// (betweenness backward passes), uploaded on first use.
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

// phast_trees for a validated handle on the current device
int trees(phast_ctx* h, const uint32_t* sources, uint32_t k, uint32_t* dist, cudaStream_t st) {
    const uint32_t kp = kpad(k);
    Sources S;
    int rc = map_sources(h, sources, k, kp, S);
    if (rc) return rc;
    if (kp == k) {
        QueryOut o{dist};
        return run_query(h, S, k, o, st);
    }
    // padded: sweep kp trees into this slot's scratch, then copy the k columns out
    const uint32_t s = h->slot_next;
    if (cudaStreamWaitEvent(st, h->slot_free[s], 0) != cudaSuccess) return PHAST_ECUDA;   // scratch reuse
    if ((rc = grow(&h->pad[s], &h->pad_elems[s], (size_t)h->n * kp))) return rc;
    QueryOut o{h->pad[s]};
    o.compact_to = dist;
    o.kc = k;
    return run_query(h, S, kp, o, st);
}

int check_handle(const phast_ctx* h) {
    if (!h) return PHAST_EINVAL;
    if (h->device < 0) return PHAST_ESTATE;
    return PHAST_OK;
}

// diameter batches on up to SLOTS library streams: lanes whose label buffers fit 2 GiB
uint32_t diameter_lanes(const phast_ctx* h, uint32_t kp, uint64_t nb) {
    const uint64_t bytes = (uint64_t)h->n * kp * 4;
    uint64_t lanes = std::max<uint64_t>(1, (2ull << 30) / std::max<uint64_t>(bytes, 1));
    return (uint32_t)std::min<uint64_t>({lanes, (uint64_t)SLOTS, nb});
}

int diameter(phast_ctx* h, const uint32_t* sources, uint64_t count, uint32_t k_batch, uint32_t* max_dev,
             uint32_t* bm, cudaStream_t st) {
    const uint32_t kp = kpad(k_batch);
    const uint64_t nb = (count + k_batch - 1) / k_batch;
    const uint32_t nl = diameter_lanes(h, kp, nb);
    int rc;
    for (uint32_t l = 0; l < nl; l++)
        if ((rc = grow(&h->lane_dist[l], &h->lane_elems[l], (size_t)h->n * kp))) return rc;
    if (cudaMemsetAsync(bm, 0, nb * 4, st) != cudaSuccess) return PHAST_ECUDA;
    // fork: every lane starts after the work queued on st so far
    if (cudaEventRecord(h->fork_ev, st) != cudaSuccess) return PHAST_ECUDA;
    for (uint32_t l = 0; l < nl; l++)
        if (cudaStreamWaitEvent(h->lane[l], h->fork_ev, 0) != cudaSuccess) return PHAST_ECUDA;
    for (uint64_t b = 0; b < nb; b++) {
        Sources S;
        const uint64_t base = b * k_batch;
        for (uint32_t i = 0; i < kp; i++) {
            const uint64_t idx = i < k_batch && base + i < count ? base + i : base;   // pad: duplicates
            S.s[i] = h->L.perm[sources[idx]];
        }
        for (uint32_t i = kp; i < KMAX; i++) S.s[i] = 0;
        const uint32_t l = (uint32_t)(b % nl);
        QueryOut o{h->lane_dist[l]};
        o.diam = bm + b;
        if ((rc = run_query(h, S, kp, o, h->lane[l]))) return rc;
    }
    // join
    for (uint32_t l = 0; l < nl; l++)
        if (cudaEventRecord(h->lane_ev[l], h->lane[l]) != cudaSuccess || cudaStreamWaitEvent(st, h->lane_ev[l], 0) != cudaSuccess)
            return PHAST_ECUDA;
    if (launch_max_reduce(bm, (uint32_t)nb, max_dev, st) != cudaSuccess) return PHAST_ECUDA;
    return PHAST_OK;
}

int batch_max_buffer(phast_ctx* h, uint64_t nb, uint32_t** bm) {
    int rc = grow(&h->batch_max_scratch, &h->batch_max_elems, nb);
    *bm = h->batch_max_scratch;
    return rc;
}

}  // namespace

extern "C" {

int phast_build(uint32_t n, const uint64_t* first, const uint32_t* head, const uint32_t* len, const phast_opts* opts,
                phast_ctx** out) {
    if (!out) return PHAST_EINVAL;
    *out = nullptr;
    int rc = validate_csr(n, first, head, len);
    if (rc) return rc;
    const uint32_t flags = opts ? opts->flags : 0u;
    if (flags & ~(PHAST_FLAG_HOST_ONLY | PHAST_FLAG_LEVEL_LAYOUT | PHAST_FLAG_BFS_IN_LEVEL | PHAST_FLAG_NO_BANDS))
        return PHAST_EINVAL;
    std::unique_ptr<phast_ctx> h(new (std::nothrow) phast_ctx());
    if (!h) return PHAST_ENOMEM;
    try {
        ChResult R;
        rc = ch_build(n, first, head, len, to_ch_options(opts), R);
        if (rc) return rc;
        h->n = n;
        h->m = first[n];
        h->shortcuts = R.shortcuts;
        h->rounds = R.rounds;
        const uint32_t mode = ((flags & PHAST_FLAG_LEVEL_LAYOUT) && !(flags & PHAST_FLAG_BFS_IN_LEVEL))
                                  ? LAYOUT_LEVELS
                              : (flags & PHAST_FLAG_NO_BANDS) ? LAYOUT_LEVELS_BFS
                                                              : LAYOUT_LEVELS_BANDS;
        rc = layout_build(R, first, head, mode, h->L);
        h->build_seconds = R.seconds;
        if (rc) return rc;
        rc = build_in_csr(h->L, n, first, head, len);
        if (rc) return rc;
        count_tails(h.get());
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

int phast_configure(phast_ctx* h, const phast_query_opts* q) {
    int rc = check_handle(h);
    if (rc) return rc;
    phast_query_opts nq = q ? *q : phast_query_opts{0, 0, 0, 0, 0, 0, 0};
    if (nq.band_threads && nq.band_threads != 128 && nq.band_threads != 256) return PHAST_EINVAL;
    if (!(nq.band_variant == 0 || nq.band_variant == 1 || nq.band_variant == 4 || nq.band_variant == 5 ||
          nq.band_variant == 13))
        return PHAST_EINVAL;
    const uint32_t known = PHAST_Q_NO_FUSED | PHAST_Q_NO_TOP | PHAST_Q_HYBRID_ON | PHAST_Q_HYBRID_OFF | PHAST_Q_NO_MULTI |
                           PHAST_Q_NO_BANDS;
    if ((nq.flags & ~known) || ((nq.flags & PHAST_Q_HYBRID_ON) && (nq.flags & PHAST_Q_HYBRID_OFF)))
        return PHAST_EINVAL;
    DeviceGuard dg(h->device);
    if (!dg.ok || cudaDeviceSynchronize() != cudaSuccess) { cudaGetLastError(); return PHAST_ECUDA; }
    free_tops(h);
    free_seeds(h);
    h->q = nq;
    return alloc_seeds(h);
}

int phast_trees(phast_ctx* h, const uint32_t* sources, uint32_t k, uint32_t* dist, void* stream) {
    int rc = check_handle(h);
    if (rc) return rc;
    if (!sources || !dist || !k_valid(k)) return PHAST_EINVAL;
    if (k % 4 == 0 && kpad(k) == k && ((uintptr_t)dist & 15)) return PHAST_EINVAL;
    if (((uintptr_t)dist & 3)) return PHAST_EINVAL;
    DeviceGuard dg(h->device);
    if (!dg.ok) return PHAST_ECUDA;
    return trees(h, sources, k, dist, (cudaStream_t)stream);
}

int phast_sync(phast_ctx* h, void* stream) {
    int rc = check_handle(h);
    if (rc) return rc;
    DeviceGuard dg(h->device);
    cudaError_t ce = cudaStreamSynchronize((cudaStream_t)stream);
    if (ce != cudaSuccess) {
        cudaGetLastError();
        return PHAST_ECUDA;
    }
    uint32_t err = 0;
    if (cudaMemcpy(&err, h->g.err, 4, cudaMemcpyDeviceToHost) != cudaSuccess) return PHAST_ECUDA;
    if (err) {
        cudaMemset(h->g.err, 0, 4);
        return (err & 1u) ? PHAST_ERANGE : PHAST_ECUDA;   // bit 0: over capacity / over 2^53
    }
    return PHAST_OK;
}

int phast_trees_host(phast_ctx* h, const uint32_t* sources, uint32_t k, uint32_t* host_dist, void* stream) {
    int rc = check_handle(h);
    if (rc) return rc;
    if (!sources || !host_dist || !k_valid(k)) return PHAST_EINVAL;
    DeviceGuard dg(h->device);
    if (!dg.ok) return PHAST_ECUDA;
    const size_t elems = (size_t)h->n * k;
    cudaStream_t st = (cudaStream_t)stream;
    if ((rc = grow(&h->host_scratch, &h->host_elems, elems))) return rc;
    if ((rc = trees(h, sources, k, h->host_scratch, st))) return rc;
    if (cudaMemcpyAsync(host_dist, h->host_scratch, elems * 4, cudaMemcpyDeviceToHost, st) != cudaSuccess)
        return PHAST_ECUDA;
    return phast_sync(h, stream);
}

int phast_parents(phast_ctx* h, const uint32_t* sources, uint32_t k, const uint32_t* dist, uint32_t* parent,
                  void* stream) {
    int rc = check_handle(h);
    if (rc) return rc;
    if (!sources || !dist || !parent || !k_valid(k)) return PHAST_EINVAL;
    if (k % 4 == 0 && kpad(k) == k && (((uintptr_t)dist & 15) || ((uintptr_t)parent & 15))) return PHAST_EINVAL;
    if (h->L.in_first.size() != (size_t)h->n + 1) return PHAST_ESTATE;
    Sources S;
    if ((rc = map_sources(h, sources, k, k, S))) return rc;
    DeviceGuard dg(h->device);
    if (!dg.ok) return PHAST_ECUDA;
    if ((rc = ensure_in_csr(h))) return rc;
    if (launch_parents(h->d_in_first, h->d_in_arc, h->n, S, k, dist, parent, (cudaStream_t)stream) != cudaSuccess)
        return PHAST_ECUDA;
    return PHAST_OK;
}

int phast_parents_ch(phast_ctx* h, const uint32_t* sources, uint32_t k, const uint32_t* dist, uint32_t* parent,
                     void* stream) {
    int rc = check_handle(h);
    if (rc) return rc;
    if (!sources || !dist || !parent || !k_valid(k)) return PHAST_EINVAL;
    if (k % 4 == 0 && kpad(k) == k && (((uintptr_t)dist & 15) || ((uintptr_t)parent & 15))) return PHAST_EINVAL;
    Sources S;
    if ((rc = map_sources(h, sources, k, k, S))) return rc;
    DeviceGuard dg(h->device);
    if (!dg.ok) return PHAST_ECUDA;
    if (!h->d_upall_first) {
        std::vector<uint32_t> f;
        std::vector<Arc> arc;
        if (!upin_csr(h->L, h->n, 0xFFFFFFFFu, f, arc) || !upload_csr(f, arc, &h->d_upall_first, &h->d_upall_arc))
            return PHAST_ENOMEM;
    }
    if (launch_parents_ch(h->g.dn_first, h->g.dn_arc, h->d_upall_first, h->d_upall_arc, h->n, S, k, dist, parent,
                          (cudaStream_t)stream) != cudaSuccess)
        return PHAST_ECUDA;
    return PHAST_OK;
}

int phast_diameter(phast_ctx* h, const uint32_t* sources, uint64_t count, uint32_t k_batch, uint32_t* max_dev,
                   uint32_t* batch_max_dev, void* stream) {
    int rc = check_handle(h);
    if (rc) return rc;
    if (!sources || !max_dev || count == 0 || !k_valid(k_batch)) return PHAST_EINVAL;
    for (uint64_t i = 0; i < count; i++)
        if (sources[i] >= h->n) return PHAST_ERANGE;
    const uint64_t nb = (count + k_batch - 1) / k_batch;
    if (nb > 0xFFFFFFFFull) return PHAST_ERANGE;
    DeviceGuard dg(h->device);
    if (!dg.ok) return PHAST_ECUDA;
    uint32_t* bm = batch_max_dev;
    if (!bm && (rc = batch_max_buffer(h, nb, &bm))) return rc;
    return diameter(h, sources, count, k_batch, max_dev, bm, (cudaStream_t)stream);
}

int phast_diameter_witness(phast_ctx* h, const uint32_t* sources, uint64_t count, uint32_t k_batch, uint32_t* out,
                           void* stream) {
    int rc = check_handle(h);
    if (rc) return rc;
    if (!sources || !out || count == 0 || !k_valid(k_batch)) return PHAST_EINVAL;
    for (uint64_t i = 0; i < count; i++)
        if (sources[i] >= h->n) return PHAST_ERANGE;
    const uint32_t kp = kpad(k_batch);
    const uint64_t nb = (count + k_batch - 1) / k_batch;
    if (nb > 0xFFFFFFFFull || (uint64_t)h->n * kp >= 0xFFFFFFFFull) return PHAST_ERANGE;
    DeviceGuard dg(h->device);
    if (!dg.ok) return PHAST_ECUDA;
    cudaStream_t st = (cudaStream_t)stream;
    uint32_t* bm = nullptr;
    if ((rc = batch_max_buffer(h, nb, &bm))) return rc;
    if (!h->wit && (rc = dmalloc(&h->wit, 4))) return rc;
    if ((rc = diameter(h, sources, count, k_batch, h->wit, bm, st))) return rc;
    if ((rc = phast_sync(h, stream))) return rc;
    std::vector<uint32_t> hb(nb);
    uint32_t D = 0;
    if (cudaMemcpy(&D, h->wit, 4, cudaMemcpyDeviceToHost) != cudaSuccess ||
        cudaMemcpy(hb.data(), bm, nb * 4, cudaMemcpyDeviceToHost) != cudaSuccess)
        return PHAST_ECUDA;
    out[0] = D;
    out[1] = out[2] = sources[0];
    if (D == 0) return PHAST_OK;
    uint64_t b = 0;
    while (b < nb && hb[b] != D) b++;
    if (b == nb) return PHAST_EINTERNAL;
    // the arg-max batch again, as trees (rows of every level stored), then an on-device argmax
    const uint64_t base = b * k_batch;
    const uint32_t kv = (uint32_t)std::min<uint64_t>(k_batch, count - base);
    std::vector<uint32_t> bs(sources + base, sources + base + kv);
    if ((rc = grow(&h->lane_dist[0], &h->lane_elems[0], (size_t)h->n * kp))) return rc;
    Sources S;
    if ((rc = map_sources(h, bs.data(), kv, kp, S))) return rc;
    QueryOut o{h->lane_dist[0]};
    unsigned long long* key = reinterpret_cast<unsigned long long*>(h->wit + 2);
    if ((rc = run_query(h, S, kp, o, st))) return rc;
    if (cudaMemsetAsync(key, 0, 8, st) != cudaSuccess ||
        launch_argmax(h->lane_dist[0], h->n, kp, kv, key, st) != cudaSuccess)
        return PHAST_ECUDA;
    if ((rc = phast_sync(h, stream))) return rc;
    unsigned long long hk = 0;
    if (cudaMemcpy(&hk, key, 8, cudaMemcpyDeviceToHost) != cudaSuccess) return PHAST_ECUDA;
    if ((uint32_t)(hk >> 32) != D) return PHAST_EINTERNAL;
    const uint32_t item = 0xFFFFFFFFu - (uint32_t)(hk & 0xFFFFFFFFull);
    out[1] = bs[item % kp];
    out[2] = h->L.iperm[item / kp];
    return PHAST_OK;
}

}  // extern "C"

namespace {
// NEXT-3 driver shared by phast_betweenness (out = double cb[n]) and phast_reach
// (out = uint32 r[n]): per batch the trees, then the Kahn-order passes, then the accumulation.
int centrality(phast_ctx* h, const uint32_t* sources, uint64_t count, uint32_t k_batch, void* out, bool reach,
               void* stream) {
    int rc = check_handle(h);
    if (rc) return rc;
    if (!sources || !out || count == 0 || !k_valid(k_batch)) return PHAST_EINVAL;
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
    const uint32_t n = h->n, k = kpad(k_batch);   // a batch is k sources (k_batch rounded up)
    const uint64_t nk = (uint64_t)n * k;
    if (nk >= 0xFFFFFFFFull) return PHAST_ERANGE;   // items are 32-bit
    if ((rc = ensure_in_csr(h)) || (rc = ensure_out_csr(h))) return rc;
    // B batches share each chain of Kahn passes: as many as 40 n k bytes each fit half
    // the free memory, at most 64 GiB and 32 batches (C2, k 64: 32 batches = 82 GB;
    // larger groups were measured slower per source: the passes turn DRAM-bound), B n k < 2^32
    size_t free_b = 0, total_b = 0;
    if (cudaMemGetInfo(&free_b, &total_b) != cudaSuccess) { cudaGetLastError(); free_b = 1ull << 32; }
    const uint64_t nbatches = (count + k - 1) / k;
    const uint64_t budget = std::min<uint64_t>(free_b / 2 + (uint64_t)h->bc_elems * 40, 64ull << 30);
    uint64_t B = std::max<uint64_t>(1, budget / (40 * nk));
    B = std::min<uint64_t>({B, 32, nbatches, 0xFFFFFFFEull / nk});
    const size_t elems = (size_t)(B * nk);
    constexpr uint32_t R = 30;   // passes per graph launch / host convergence check (multiple of 6)
    if (!h->bc_changed) {
        if ((rc = dmalloc(&h->bc_changed, R)) || (rc = dmalloc(&h->bc_qs, 3))) return rc;
        if (cudaMallocHost(&h->bc_changed_host, R * 4) != cudaSuccess) {
            cudaGetLastError();
            return PHAST_ENOMEM;
        }
    }
    if (h->bc_elems < elems) {
        cudaFree(h->bc_sigma); cudaFree(h->bc_delta); cudaFree(h->bc_q); cudaFree(h->bc_dist); cudaFree(h->bc_src);
        h->bc_sigma = h->bc_delta = nullptr;
        h->bc_q = h->bc_dist = h->bc_src = nullptr;
        h->bc_elems = 0;
        if ((rc = dmalloc(&h->bc_sigma, elems)) || (rc = dmalloc(&h->bc_delta, elems)) ||
            (rc = dmalloc(&h->bc_q, 5 * elems)) || (rc = dmalloc(&h->bc_dist, elems)) ||
            (rc = dmalloc(&h->bc_src, (size_t)B * k)))
            return rc;
        h->bc_elems = elems;
    }
    if (cudaMemsetAsync(out, 0, (size_t)n * (reach ? 4 : 8), st) != cudaSuccess) return PHAST_ECUDA;
    // Kahn order (next.cu): the count kernel fills queue 0; pass p reads queue p%2 with
    // size qs[p%3], appends to queue (p+1)%2 with qs[(p+1)%3], zeroes qs[(p+2)%3]; stop
    // after a pass that readied nothing (<= hop depth of the tight DAG + 1 passes)
    uint32_t* d = h->bc_dist;
    const BcGraph G{h->d_in_first, h->d_in_arc, h->d_out_first, h->d_out_arc, h->g.err};
    uint32_t* qbuf[2] = {h->bc_q, h->bc_q + elems};
    uint32_t* cnt = h->bc_q + 2 * elems;
    uint32_t* mask_in = h->bc_q + 3 * elems;    // tight-arc masks (the forward count computes both)
    uint32_t* mask_out = h->bc_q + 4 * elems;
    // R passes (+ clearing the change words before, reading them back after) are one CUDA
    // graph, captured once per group size and direction on a private stream (the caller's
    // stream may be the legacy default stream, which cannot be captured); R is a multiple
    // of 6, so every chunk starts with the same queue/counter rotation.
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
    uint32_t total = 0;   // items of the current group (B' batches)
    uint32_t graph_total = 0;
    auto kahn = [&](int which, int backward, auto pass) -> int {
        if (execs[which] && graph_total != total) {   // a smaller last group: re-capture
            cudaGraphExecDestroy(execs[which]);
            execs[which] = nullptr;
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
            launch_bc_count(G, d, (uint32_t)nk, k, total, backward, cnt, mask_in, mask_out, qbuf[0], h->bc_qs, gs) !=
                cudaSuccess)
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
    std::vector<uint32_t> gsrc((size_t)B * k);
    for (uint64_t base = 0; base < count; base += B * k) {
        // a group: B' batches of k trees, labels into [b][n][k]
        const uint64_t left = count - base;
        const uint32_t Bg = (uint32_t)std::min<uint64_t>(B, (left + k - 1) / k);
        const uint32_t valid = (uint32_t)std::min<uint64_t>(left, (uint64_t)Bg * k);
        total = (uint32_t)(Bg * nk);
        for (uint32_t b = 0; b < Bg; b++) {
            const uint32_t kv = (uint32_t)std::min<uint64_t>(k, valid - (uint64_t)b * k);
            Sources S;
            if ((rc = map_sources(h, sources + base + (uint64_t)b * k, kv, k, S))) return rc;
            for (uint32_t i = 0; i < k; i++) gsrc[(size_t)b * k + i] = S.s[i];
            QueryOut o{d + (size_t)b * nk};
            if ((rc = run_query(h, S, k, o, st))) return rc;
        }
        if (cudaMemcpyAsync(h->bc_src, gsrc.data(), (size_t)Bg * k * 4, cudaMemcpyHostToDevice, st) != cudaSuccess)
            return PHAST_ECUDA;
        if (reach) {
            if (cudaMemsetAsync(hgt, 0, (size_t)total * 4, st) != cudaSuccess) return PHAST_ECUDA;
            // the masks come from the forward count: run it (no passes) before the height
            if (cudaEventRecord(h->bc_ev, st) != cudaSuccess || cudaStreamWaitEvent(gs, h->bc_ev, 0) != cudaSuccess ||
                cudaMemsetAsync(h->bc_qs, 0, 12, gs) != cudaSuccess ||
                launch_bc_count(G, d, (uint32_t)nk, k, total, 0, cnt, mask_in, mask_out, qbuf[0], h->bc_qs, gs) !=
                    cudaSuccess ||
                cudaEventRecord(h->bc_ev, gs) != cudaSuccess || cudaStreamWaitEvent(st, h->bc_ev, 0) != cudaSuccess)
                return PHAST_ECUDA;
            rc = kahn(2, 1, [&](const BcQueue& Q, uint32_t* ch, cudaStream_t s2) {
                return launch_bc_back(G, d, nullptr, hgt, (uint32_t)nk, k, total, mask_in, mask_out, 1, Q, ch, s2);
            });
            if (rc) return rc;
            graph_total = total;
            if (launch_reach_accum(d, hgt, (uint32_t*)out, n, k, valid, st) != cudaSuccess) return PHAST_ECUDA;
            continue;
        }
        if (cudaMemsetAsync(h->bc_sigma, 0, (size_t)total * 8, st) != cudaSuccess ||
            cudaMemsetAsync(h->bc_delta, 0, (size_t)total * 8, st) != cudaSuccess)
            return PHAST_ECUDA;
        rc = kahn(0, 0, [&](const BcQueue& Q, uint32_t* ch, cudaStream_t s2) {
            return launch_bc_sigma(G, d, h->bc_sigma, (uint32_t)nk, k, total, mask_in, mask_out, Q, ch, s2);
        });
        if (rc) return rc;
        rc = kahn(1, 1, [&](const BcQueue& Q, uint32_t* ch, cudaStream_t s2) {
            return launch_bc_back(G, d, h->bc_sigma, h->bc_delta, (uint32_t)nk, k, total, mask_in, mask_out, 0, Q, ch,
                                  s2);
        });
        if (rc) return rc;
        graph_total = total;
        if (launch_bc_accum(h->bc_delta, (double*)out, n, k, valid, h->bc_src, st) != cudaSuccess) return PHAST_ECUDA;
    }
    return phast_sync(h, stream);
}

// upward search space of internal id s: the vertices reachable from s in G-up (the
// search runs to exhaustion, §III), counted with an epoch-stamped mark
uint32_t up_space(const Layout& L, uint32_t s, std::vector<uint32_t>& mark, uint32_t epoch,
                  std::vector<uint32_t>& stack) {
    uint32_t cnt = 0;
    stack.clear();
    stack.push_back(s);
    mark[s] = epoch;
    while (!stack.empty()) {
        const uint32_t v = stack.back();
        stack.pop_back();
        cnt++;
        for (uint32_t e = L.up_first[v]; e < L.up_first[v + 1]; e++) {
            const uint32_t w = L.up_arc[e].x;
            if (mark[w] != epoch) { mark[w] = epoch; stack.push_back(w); }
        }
    }
    return cnt;
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
    if (!h->up_stats) {   // seeded sample of sources (a fixed odd stride over the ids)
        const uint32_t n = h->n, cnt = std::min(n, UP_SAMPLE);
        std::vector<uint32_t> mark(n, 0), stack;
        double sum = 0;
        uint32_t mx = 0;
        for (uint32_t i = 0; i < cnt; i++) {
            const uint32_t s = (uint32_t)(((uint64_t)i * 2654435761ull + 12345) % n);
            const uint32_t c = up_space(h->L, s, mark, i + 1, stack);
            sum += c;
            mx = std::max(mx, c);
        }
        h->up_mean = cnt ? sum / cnt : 0.0;
        h->up_max = mx;
        h->up_samples = cnt;
        h->up_stats = true;
    }
    std::memset(o, 0, sizeof(*o));
    o->n = h->n;
    o->levels = h->L.levels;
    o->m = h->m;
    o->m_up = h->L.up_arc.size();
    o->m_down = h->L.dn_arc.size();
    o->n_tail = h->n_tail;
    o->shortcuts = h->shortcuts;
    o->rounds = h->rounds;
    o->device = h->device < 0 ? 0xFFFFFFFFu : (uint32_t)h->device;
    o->layout = h->L.mode;
    o->up_space_samples = h->up_samples;
    o->build_seconds = h->build_seconds;
    o->mean_up_space = h->up_mean;
    o->max_up_space = h->up_max;
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

int phast_bands(const phast_ctx* h, uint32_t* count, uint32_t* desc) {
    if (!h || !count) return PHAST_EINVAL;
    *count = (uint32_t)h->L.bands.size();
    if (desc)
        for (size_t b = 0; b < h->L.bands.size(); b++) {
            desc[3 * b] = h->L.bands[b].seg_lo;
            desc[3 * b + 1] = h->L.bands[b].seg_hi;
            desc[3 * b + 2] = h->L.bands[b].ngroups;
        }
    return PHAST_OK;
}

int phast_band_groups(const phast_ctx* h, uint32_t b, uint32_t* goff) {
    if (!h || !goff || b >= h->L.bands.size()) return PHAST_EINVAL;
    const auto& g = h->L.bands[b].goff;
    std::memcpy(goff, g.data(), g.size() * 4);
    return PHAST_OK;
}

int phast_schedule(phast_ctx* h, uint32_t k, uint32_t* out) {
    int rc = check_handle(h);
    if (rc) return rc;
    if (!out || !k_valid(k)) return PHAST_EINVAL;
    DeviceGuard dg(h->device);
    if (!dg.ok) return PHAST_ECUDA;
    const uint32_t kp = kpad(k);
    const phast_ctx::Top* t = get_top(h, kp);
    const uint32_t levels = (uint32_t)h->L.lvl_off.size() - 1;
    for (int i = 0; i < 6; i++) out[i] = 0;
    out[0] = t && t->a.fused ? 1u : 0u;
    out[1] = t ? t->J : 0u;
    out[2] = t ? t->a.V : 0u;
    if (out[0]) return PHAST_OK;
    std::vector<phast_ctx::BandRun>* bands = nullptr;   // the walk of run_query
    if (!(h->q.flags & PHAST_Q_NO_BANDS) && !h->L.bands.empty() && (rc = get_bands(h, kp, &bands))) return rc;
    size_t bi = 0;
    for (uint32_t j = t ? t->J : 0u; j < levels;) {
        while (bands && bi < bands->size() && (*bands)[bi].seg_lo < j) bi++;
        if (bands && bi < bands->size() && (*bands)[bi].seg_lo == j) {
            out[4]++;
            out[5] += (*bands)[bi].seg_hi - j;
            j = (*bands)[bi++].seg_hi;
        } else {
            out[3]++;
            j++;
        }
    }
    return PHAST_OK;
}

// ---------------------------------------------------------------- save / load
static const char MAGIC[8] = {'P', 'H', 'A', 'S', 'T', 'B', '2', '5'};

int phast_save(const phast_ctx* h, const char* path) {
    if (!h || !path) return PHAST_EINVAL;
    FILE* f = std::fopen(path, "wb");
    if (!f) return PHAST_EIO;
    const Layout& L = h->L;
    uint64_t hdr[10] = {h->n, L.levels, h->m, h->shortcuts, h->rounds, L.dn_arc.size(), L.up_arc.size(),
                        L.mode, 0, L.lvl_off.size()};
    auto wr = [&](const void* p, size_t sz, size_t cnt) { return std::fwrite(p, sz, cnt, f) == cnt; };
    bool ok = wr(MAGIC, 1, 8) && wr(hdr, 8, 10) && wr(&h->build_seconds, 8, 1) && wr(L.perm.data(), 4, h->n) &&
              wr(L.level.data(), 4, h->n) && wr(L.lvl_off.data(), 4, L.lvl_off.size()) &&
              wr(L.dn_first.data(), 4, L.dn_first.size()) && wr(L.up_first.data(), 4, L.up_first.size()) &&
              wr(L.dn_arc.data(), 8, L.dn_arc.size()) && wr(L.up_arc.data(), 8, L.up_arc.size());
    const uint64_t n_in = L.in_arc.size();
    ok = ok && wr(&n_in, 8, 1) && wr(L.in_first.data(), 4, L.in_first.size()) && wr(L.in_arc.data(), 8, n_in);
    const uint64_t nb = L.bands.size();
    ok = ok && wr(&nb, 8, 1);
    for (const Band& B : L.bands) {
        const uint32_t bh[3] = {B.seg_lo, B.seg_hi, B.ngroups};
        ok = ok && wr(bh, 4, 3) && wr(B.goff.data(), 4, B.goff.size());
    }
    ok = (std::fclose(f) == 0) && ok;
    return ok ? PHAST_OK : PHAST_EIO;
}

int phast_load(const char* path, uint32_t flags, phast_ctx** out) {
    if (!path || !out) return PHAST_EINVAL;
    *out = nullptr;
    if (flags & ~PHAST_FLAG_HOST_ONLY) return PHAST_EINVAL;
    FILE* f = std::fopen(path, "rb");
    if (!f) return PHAST_EIO;
    std::unique_ptr<phast_ctx> h(new (std::nothrow) phast_ctx());
    char magic[8];
    uint64_t hdr[10];
    auto rd = [&](void* p, size_t sz, size_t cnt) { return std::fread(p, sz, cnt, f) == cnt; };
    bool ok = h && rd(magic, 1, 8) && std::memcmp(magic, MAGIC, 8) == 0 && rd(hdr, 8, 10) &&
              rd(&h->build_seconds, 8, 1) && hdr[0] > 0 && hdr[0] < 0xFFFFFFFFull &&
              (hdr[7] == LAYOUT_LEVELS || hdr[7] == LAYOUT_LEVELS_BFS || hdr[7] == LAYOUT_LEVELS_BANDS) &&
              hdr[9] == hdr[1] + 1;
    if (ok) {
        Layout& L = h->L;
        try {
            h->n = (uint32_t)hdr[0]; L.levels = (uint32_t)hdr[1]; h->m = hdr[2];
            h->shortcuts = hdr[3]; h->rounds = (uint32_t)hdr[4];
            L.mode = (uint32_t)hdr[7];
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
        uint64_t nb = 0;
        ok = ok && rd(&nb, 8, 1) && nb <= L.levels;
        for (uint64_t b = 0; ok && b < nb; b++) {
            uint32_t bh[3];
            ok = rd(bh, 4, 3) && bh[0] < bh[1] && bh[1] <= L.levels && bh[2] <= h->n;
            if (!ok) break;
            Band B;
            B.seg_lo = bh[0]; B.seg_hi = bh[1]; B.ngroups = bh[2];
            try {
                B.goff.resize((size_t)(B.seg_hi - B.seg_lo) * (B.ngroups + 1));
            } catch (const std::bad_alloc&) {
                std::fclose(f);
                return PHAST_ENOMEM;
            }
            ok = rd(B.goff.data(), 4, B.goff.size());
            L.bands.push_back(std::move(B));
        }
    }
    std::fclose(f);
    if (!ok || check_bands(h->L) != 0) return PHAST_EIO;
    for (uint32_t v = 0; v < h->n; v++) {
        if (h->L.perm[v] >= h->n) return PHAST_EIO;
        h->L.iperm[h->L.perm[v]] = v;
    }
    count_tails(h.get());
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
    int rc = check_handle(h);
    if (rc) return rc;
    if (enable) h->ev_used = 0;
    h->timing = enable != 0;
    return PHAST_OK;
}

int phast_timing_read(phast_ctx* h, double* ms_up, double* ms_sweep, uint64_t* batches) {
    if (!ms_up || !ms_sweep || !batches) return PHAST_EINVAL;
    int rc = check_handle(h);
    if (rc) return rc;
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

int phast_probe(phast_ctx* h, int kind, const uint32_t* sources, uint32_t k, uint32_t* dist, void* stream) {
    int rc = check_handle(h);
    if (rc) return rc;
    if (!dist || !k_valid(k) || kpad(k) != k || (kind != 0 && kind != 1) || (kind == 1 && !sources)) return PHAST_EINVAL;
    if (k % 4 == 0 && ((uintptr_t)dist & 15)) return PHAST_EINVAL;
    DeviceGuard dg(h->device);
    if (!dg.ok) return PHAST_ECUDA;
    cudaStream_t st = (cudaStream_t)stream;
    if (kind == 0) return launch_probe_stream(h->g, k, dist, st) == cudaSuccess ? PHAST_OK : PHAST_ECUDA;
    Sources S;
    if ((rc = map_sources(h, sources, k, k, S))) return rc;
    QueryOut o{dist};
    o.nogather = true;
    return run_query(h, S, k, o, st);
}

uint64_t phast_launch_count(void) { return launches(); }

}  // extern "C"
