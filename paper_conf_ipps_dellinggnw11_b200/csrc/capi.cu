// capi.cu -- the C ABI of include/phast.h: handle lifetime, validation, layout
// (renumbering by level), device image upload, and query orchestration.
//
// Layout:
//   internal ids sorted by (level descending, original id ascending): "We assign
//   lower IDs to vertices at higher levels; within each level, we keep the DFS
//   order" (§IV-A; the generator's ids are the DFS order).  Then the
//   sweep is "a simple linear sweep in increasing order of IDs", and every level is
//   one contiguous id range [lvl_off[j], lvl_off[j+1]).
//   G-down: in-arcs by head, {tail, len} (§IV-A), sentinel dn_first[n].
//   G-up:   out-arcs by tail, {head, len}.
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

using namespace phast;

struct phast_ctx {
    uint32_t n = 0, levels = 0;
    uint64_t m = 0, shortcuts = 0;
    uint32_t rounds = 0;
    double build_seconds = 0;
    std::vector<uint32_t> perm;      // internal_of_original
    std::vector<uint32_t> iperm;     // original_of_internal
    std::vector<uint32_t> lvl_off;   // [levels+1], j = 0 is the top level
    std::vector<uint32_t> dn_first, up_first;
    std::vector<uint2> dn_arc, up_arc;
    // device
    int device = -1;
    DevImage g;
    uint32_t* dist_scratch = nullptr;   // diameter mode label buffer
    size_t dist_scratch_elems = 0;
    uint32_t* batch_max_scratch = nullptr;
    size_t batch_max_elems = 0;
    // persistent-sweep plans, one per k (built on first use)
    struct Plan {
        SweepPlan p;
        uint32_t epoch = 0;
        bool ok = false;
    };
    std::map<uint32_t, Plan> plans;
    std::vector<uint32_t> level_of;   // processing index of every internal id (lazy)
    int sweep_mode = 0;               // 0 = persistent, 1 = one launch per level
    // stage timing (phast_timing)
    bool timing = false;
    std::vector<cudaEvent_t> ev;     // 3 per recorded batch
    size_t ev_used = 0;
};

namespace {

constexpr uint32_t SEED_CAP = 1u << 16;   // per-source search-space capacity (global fallback)

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
    if (e != cudaSuccess) { cudaGetLastError(); *p = nullptr; return e == cudaErrorMemoryAllocation ? PHAST_ENOMEM : PHAST_ECUDA; }
    return PHAST_OK;
}

void free_device(phast_ctx* h) {
    if (h->device < 0) return;
    DeviceGuard dg(h->device);
    cudaDeviceSynchronize();
    for (auto& kv : h->plans) {
        cudaFree((void*)kv.second.p.chunk_v); cudaFree((void*)kv.second.p.chunk_meta);
        cudaFree((void*)kv.second.p.chunk_start); cudaFree((void*)kv.second.p.lvl_off);
        cudaFree(kv.second.p.level_done);
    }
    h->plans.clear();
    for (cudaEvent_t e : h->ev) cudaEventDestroy(e);
    h->ev.clear();
    h->ev_used = 0;
    cudaFree((void*)h->g.dn_first); cudaFree((void*)h->g.dn_arc);
    cudaFree((void*)h->g.up_first); cudaFree((void*)h->g.up_arc);
    cudaFree(h->g.flags); cudaFree(h->g.seed_v); cudaFree(h->g.seed_d); cudaFree(h->g.seed_cnt);
    cudaFree(h->g.gscratch); cudaFree(h->g.err);
    cudaFree(h->dist_scratch); cudaFree(h->batch_max_scratch);
    h->g = DevImage();
    h->dist_scratch = nullptr; h->batch_max_scratch = nullptr;
    h->device = -1;
}

int upload(phast_ctx* h) {
    int dev = 0;
    if (cudaGetDevice(&dev) != cudaSuccess) { cudaGetLastError(); return PHAST_ECUDA; }
    h->device = dev;
    DevImage& g = h->g;
    g.n = h->n;
    // test knobs (power of two): shrink the shared-memory table / per-source capacity to
    // exercise the global-memory fallback and the overflow error path
    uint32_t seed_cap = SEED_CAP, smem_cap = 4096;
    if (const char* e = std::getenv("PHAST_SEED_CAP")) seed_cap = std::max(16u, std::min<uint32_t>(SEED_CAP, (uint32_t)std::atoi(e)));
    if (const char* e = std::getenv("PHAST_UP_SMEM_CAP")) smem_cap = std::max(16u, std::min<uint32_t>(4096u, (uint32_t)std::atoi(e)));
    auto pow2 = [](uint32_t x) { uint32_t p = 1; while (p * 2 <= x) p *= 2; return p; };
    g.seed_cap = pow2(seed_cap);
    g.smem_cap = pow2(smem_cap);
    uint32_t *dnf, *upf;
    uint2 *dna, *upa;
    int rc;
    size_t nw = ((size_t)h->n + 31) / 32;
    if ((rc = dmalloc(&dnf, h->dn_first.size())) || (rc = dmalloc(&dna, h->dn_arc.size())) ||
        (rc = dmalloc(&upf, h->up_first.size())) || (rc = dmalloc(&upa, h->up_arc.size())) ||
        (rc = dmalloc(&g.flags, nw)) || (rc = dmalloc(&g.seed_v, (size_t)KMAX * g.seed_cap)) ||
        (rc = dmalloc(&g.seed_d, (size_t)KMAX * g.seed_cap)) || (rc = dmalloc(&g.seed_cnt, KMAX)) ||
        (rc = dmalloc(&g.gscratch, (size_t)KMAX * g.seed_cap * 5)) || (rc = dmalloc(&g.err, 1))) {
        g.dn_first = dnf; g.dn_arc = dna; g.up_first = upf; g.up_arc = upa;
        free_device(h);
        return rc;
    }
    g.dn_first = dnf; g.dn_arc = dna; g.up_first = upf; g.up_arc = upa;
    bool ok = cudaMemcpy(dnf, h->dn_first.data(), h->dn_first.size() * 4, cudaMemcpyHostToDevice) == cudaSuccess &&
              cudaMemcpy(dna, h->dn_arc.data(), h->dn_arc.size() * 8, cudaMemcpyHostToDevice) == cudaSuccess &&
              cudaMemcpy(upf, h->up_first.data(), h->up_first.size() * 4, cudaMemcpyHostToDevice) == cudaSuccess &&
              cudaMemcpy(upa, h->up_arc.data(), h->up_arc.size() * 8, cudaMemcpyHostToDevice) == cudaSuccess &&
              cudaMemset(g.flags, 0, nw * 4) == cudaSuccess && cudaMemset(g.err, 0, 4) == cudaSuccess &&
              cudaMemset(g.seed_cnt, 0, KMAX * 4) == cudaSuccess && cudaDeviceSynchronize() == cudaSuccess;
    if (!ok) { cudaGetLastError(); free_device(h); return PHAST_ECUDA; }
    return PHAST_OK;
}

// renumber by (level desc, id asc) and build the two CSRs in internal ids
int layout(phast_ctx* h, const ChResult& R) {
    const uint32_t n = R.n;
    uint32_t L = 0;
    for (uint32_t v = 0; v < n; v++) L = std::max(L, R.level[v] + 1);
    h->levels = L;
    std::vector<uint32_t> cnt(L, 0);
    for (uint32_t v = 0; v < n; v++) cnt[R.level[v]]++;
    h->lvl_off.assign(L + 1, 0);
    for (uint32_t j = 0; j < L; j++) h->lvl_off[j + 1] = h->lvl_off[j] + cnt[L - 1 - j];
    std::vector<uint32_t> pos(L);
    for (uint32_t j = 0; j < L; j++) pos[L - 1 - j] = h->lvl_off[j];
    h->perm.resize(n);
    h->iperm.resize(n);
    for (uint32_t v = 0; v < n; v++) {   // ascending original id within each level
        uint32_t r = pos[R.level[v]]++;
        h->perm[v] = r;
        h->iperm[r] = v;
    }
    uint64_t mdn = R.dn_first[n], mup = R.up_first[n];
    if (mdn >= 0xFFFFFFFFull || mup >= 0xFFFFFFFFull) return PHAST_ERANGE;
    h->dn_first.assign((size_t)n + 1, 0);
    h->up_first.assign((size_t)n + 1, 0);
    h->dn_arc.resize(mdn);
    h->up_arc.resize(mup);
    for (uint32_t r = 0; r < n; r++) {
        uint32_t v = h->iperm[r];
        h->dn_first[r + 1] = h->dn_first[r] + (uint32_t)(R.dn_first[v + 1] - R.dn_first[v]);
        h->up_first[r + 1] = h->up_first[r] + (uint32_t)(R.up_first[v + 1] - R.up_first[v]);
    }
    bool lemma_ok = true;
    for (uint32_t r = 0; r < n; r++) {
        uint32_t v = h->iperm[r];
        uint32_t p = h->dn_first[r];
        for (uint64_t e = R.dn_first[v]; e < R.dn_first[v + 1]; e++) {
            uint32_t t = R.dn_tail[e];
            // Lemma 4.1: (t, v) in A-down => L(t) > L(v)  (§IV-A)
            if (!(R.level[t] > R.level[v])) lemma_ok = false;
            h->dn_arc[p++] = make_uint2(h->perm[t], R.dn_len[e]);
        }
        std::sort(h->dn_arc.begin() + h->dn_first[r], h->dn_arc.begin() + h->dn_first[r + 1],
                  [](const uint2& a, const uint2& b) { return a.x < b.x || (a.x == b.x && a.y < b.y); });
        p = h->up_first[r];
        for (uint64_t e = R.up_first[v]; e < R.up_first[v + 1]; e++) {
            uint32_t w = R.up_head[e];
            if (!(R.level[w] > R.level[v])) lemma_ok = false;    // same rule for A-up
            h->up_arc[p++] = make_uint2(h->perm[w], R.up_len[e]);
        }
        std::sort(h->up_arc.begin() + h->up_first[r], h->up_arc.begin() + h->up_first[r + 1],
                  [](const uint2& a, const uint2& b) { return a.x < b.x || (a.x == b.x && a.y < b.y); });
    }
    return lemma_ok ? PHAST_OK : PHAST_EINTERNAL;
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
        S.s[i] = h->perm[src[i]];
    }
    for (uint32_t i = k; i < KMAX; i++) S.s[i] = 0;
    return PHAST_OK;
}

// build (once per k) the chunk table of the persistent sweep
phast_ctx::Plan* get_plan(phast_ctx* h, uint32_t k) {
    auto it = h->plans.find(k);
    if (it != h->plans.end()) return it->second.ok ? &it->second : nullptr;
    phast_ctx::Plan& P = h->plans[k];
    if (h->levels == 0 || h->levels > 65534) return nullptr;
    if (h->level_of.empty()) {
        h->level_of.resize(h->n);
        for (uint32_t j = 0; j < h->levels; j++)
            for (uint32_t v = h->lvl_off[j]; v < h->lvl_off[j + 1]; v++) h->level_of[v] = j;
    }
    const uint32_t CV = sweep_chunk_vertices(k);
    std::vector<uint32_t> cstart(h->levels + 1, 0), cv, cmeta;
    for (uint32_t j = 0; j < h->levels; j++) {
        cstart[j] = (uint32_t)cv.size();
        for (uint32_t vb = h->lvl_off[j]; vb < h->lvl_off[j + 1]; vb += CV) {
            uint32_t ve = std::min(vb + CV, h->lvl_off[j + 1]);
            int D = -1;
            for (uint32_t e = h->dn_first[vb]; e < h->dn_first[ve]; e++)
                D = std::max(D, (int)h->level_of[h->dn_arc[e].x]);
            if (D >= (int)j) return nullptr;                      // would violate Lemma 4.1
            cv.push_back(vb);
            cmeta.push_back((j << 16) | (uint32_t)(D + 1));
        }
    }
    cstart[h->levels] = (uint32_t)cv.size();
    int occ = std::min(sweep_blocks_per_sm(k, false), sweep_blocks_per_sm(k, true));
    SweepPlan& p = P.p;
    p.k = k;
    p.nchunks = (uint32_t)cv.size();
    p.levels = h->levels;
    p.grid = (uint32_t)std::max(1, occ * num_sms());
    p.chunk_vertices = CV;
    uint32_t *a, *b, *c, *d, *e;
    if (dmalloc(&a, cv.size()) || dmalloc(&b, cmeta.size()) || dmalloc(&c, cstart.size()) ||
        dmalloc(&d, h->lvl_off.size()) || dmalloc(&e, h->levels))
        return nullptr;
    p.chunk_v = a; p.chunk_meta = b; p.chunk_start = c; p.lvl_off = d; p.level_done = e;
    if (cudaMemcpy(a, cv.data(), cv.size() * 4, cudaMemcpyHostToDevice) != cudaSuccess ||
        cudaMemcpy(b, cmeta.data(), cmeta.size() * 4, cudaMemcpyHostToDevice) != cudaSuccess ||
        cudaMemcpy(c, cstart.data(), cstart.size() * 4, cudaMemcpyHostToDevice) != cudaSuccess ||
        cudaMemcpy(d, h->lvl_off.data(), h->lvl_off.size() * 4, cudaMemcpyHostToDevice) != cudaSuccess ||
        cudaMemset(e, 0, h->levels * 4) != cudaSuccess) {
        cudaGetLastError();
        return nullptr;
    }
    P.ok = true;
    return &P;
}

// one full query (a1-a3) for k mapped sources; diam != nullptr -> fused max, no level-0 stores
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

int run_query(phast_ctx* h, const Sources& S, uint32_t k, uint32_t* dist, uint32_t* diam, cudaStream_t st) {
    cudaError_t e;
    cudaEvent_t e0 = nullptr, e1 = nullptr, e2 = nullptr;
    if (h->timing && h->ev_used + 3 <= 3 * MAX_TIMED_BATCHES) {
        e0 = timing_event(h); e1 = timing_event(h); e2 = timing_event(h);
        if (!e0 || !e1 || !e2) return PHAST_ECUDA;
        cudaEventRecord(e0, st);
    }
    if ((e = launch_upward(h->g, S, k, dist, st)) != cudaSuccess) return PHAST_ECUDA;
    if ((e = launch_scatter(h->g, k, dist, st)) != cudaSuccess) return PHAST_ECUDA;
    if (e1) cudaEventRecord(e1, st);
    phast_ctx::Plan* plan = h->sweep_mode == 0 ? get_plan(h, k) : nullptr;
    if (plan) {                          // a3+a4: one persistent launch, dataflow over levels
        if ((uint64_t)(plan->epoch + 1) * plan->p.grid >= 0x7FFFFFFFull) {
            if (cudaMemsetAsync(plan->p.level_done, 0, plan->p.levels * 4, st) != cudaSuccess) return PHAST_ECUDA;
            plan->epoch = 0;
        }
        plan->epoch++;
        if (launch_sweep_persistent(h->g, plan->p, plan->epoch, dist, diam, st) != cudaSuccess) return PHAST_ECUDA;
    } else {                             // one launch per level (§VI)
        for (uint32_t j = 0; j < h->levels; j++) {
            bool last = (j + 1 == h->levels);
            bool store = !(diam && last);   // level-0 rows are never read again (diameter mode)
            e = launch_sweep_level(h->g, k, h->lvl_off[j], h->lvl_off[j + 1], dist, diam, store, last, st);
            if (e != cudaSuccess) return PHAST_ECUDA;
        }
    }
    if ((e = launch_clear_flags(h->g, k, st)) != cudaSuccess) return PHAST_ECUDA;
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

}  // namespace

extern "C" {

int phast_build(uint32_t n, const uint64_t* first, const uint32_t* head, const uint32_t* len,
                const phast_opts* opts, phast_ctx** out) {
    if (!out) return PHAST_EINVAL;
    *out = nullptr;
    int rc = validate_csr(n, first, head, len);
    if (rc) return rc;
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
        h->build_seconds = R.seconds;
        rc = layout(h.get(), R);
        if (rc) return rc;
    } catch (const std::bad_alloc&) {
        return PHAST_ENOMEM;
    }
    if (!(opts && (opts->flags & PHAST_FLAG_HOST_ONLY))) {
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
    if (cudaStreamSynchronize((cudaStream_t)stream) != cudaSuccess) { cudaGetLastError(); return PHAST_ECUDA; }
    uint32_t err = 0;
    if (cudaMemcpy(&err, h->g.err, 4, cudaMemcpyDeviceToHost) != cudaSuccess) return PHAST_ECUDA;
    if (err) {
        cudaMemset(h->g.err, 0, 4);
        return PHAST_ERANGE;
    }
    return PHAST_OK;
}

int phast_trees_host(phast_ctx* h, const uint32_t* sources, uint32_t k, uint32_t* host_dist, void* stream) {
    if (!h || !sources || !host_dist || !k_ok(k)) return PHAST_EINVAL;
    if (h->device < 0) return PHAST_ESTATE;
    DeviceGuard dg(h->device);
    size_t elems = (size_t)h->n * k;
    if (h->dist_scratch_elems < elems) {
        cudaFree(h->dist_scratch);
        h->dist_scratch = nullptr;
        h->dist_scratch_elems = 0;
        int rc = dmalloc(&h->dist_scratch, elems);
        if (rc) return rc;
        h->dist_scratch_elems = elems;
    }
    int rc = phast_trees(h, sources, k, h->dist_scratch, stream);
    if (rc) return rc;
    cudaStream_t st = (cudaStream_t)stream;
    if (cudaMemcpyAsync(host_dist, h->dist_scratch, elems * 4, cudaMemcpyDeviceToHost, st) != cudaSuccess)
        return PHAST_ECUDA;
    return phast_sync(h, stream);
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
    size_t elems = (size_t)h->n * k_batch;
    if (h->dist_scratch_elems < elems) {
        cudaFree(h->dist_scratch);
        h->dist_scratch = nullptr;
        h->dist_scratch_elems = 0;
        int rc = dmalloc(&h->dist_scratch, elems);
        if (rc) return rc;
        h->dist_scratch_elems = elems;
    }
    uint64_t nb = (count + k_batch - 1) / k_batch;
    if (nb > 0xFFFFFFFFull) return PHAST_ERANGE;
    uint32_t* bm = batch_max_dev;
    if (!bm) {
        if (h->batch_max_elems < nb) {
            cudaFree(h->batch_max_scratch);
            h->batch_max_scratch = nullptr;
            h->batch_max_elems = 0;
            int rc = dmalloc(&h->batch_max_scratch, nb);
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
            S.s[i] = h->perm[sources[idx]];
        }
        int rc = run_query(h, S, k_batch, h->dist_scratch, bm + b, st);
        if (rc) return rc;
    }
    if (launch_max_reduce(bm, (uint32_t)nb, max_dev, st) != cudaSuccess) return PHAST_ECUDA;
    return PHAST_OK;
}

int phast_info(const phast_ctx* h, phast_info_t* o) {
    if (!h || !o) return PHAST_EINVAL;
    std::memset(o, 0, sizeof(*o));
    o->n = h->n;
    o->levels = h->levels;
    o->m = h->m;
    o->m_up = h->up_arc.size();
    o->m_down = h->dn_arc.size();
    std::vector<uint8_t> is_tail(h->n, 0);
    for (const uint2& a : h->dn_arc) is_tail[a.x] = 1;
    uint64_t nt = 0;
    for (uint8_t t : is_tail) nt += t;
    o->n_tail = nt;
    o->shortcuts = h->shortcuts;
    o->rounds = h->rounds;
    o->device = h->device < 0 ? 0xFFFFFFFFu : (uint32_t)h->device;
    o->build_seconds = h->build_seconds;
    return PHAST_OK;
}

int phast_level_sizes(const phast_ctx* h, uint32_t* out) {
    if (!h || !out) return PHAST_EINVAL;
    for (uint32_t j = 0; j < h->levels; j++) out[h->levels - 1 - j] = h->lvl_off[j + 1] - h->lvl_off[j];
    return PHAST_OK;
}

int phast_order(const phast_ctx* h, uint32_t* o) {
    if (!h || !o) return PHAST_EINVAL;
    std::memcpy(o, h->perm.data(), (size_t)h->n * 4);
    return PHAST_OK;
}

int phast_export(const phast_ctx* h, uint32_t* lvl_off, uint32_t* dn_first, uint32_t* dn_tail, uint32_t* dn_len,
                 uint32_t* up_first, uint32_t* up_head, uint32_t* up_len) {
    if (!h) return PHAST_EINVAL;
    if (lvl_off) std::memcpy(lvl_off, h->lvl_off.data(), h->lvl_off.size() * 4);
    if (dn_first) std::memcpy(dn_first, h->dn_first.data(), h->dn_first.size() * 4);
    if (up_first) std::memcpy(up_first, h->up_first.data(), h->up_first.size() * 4);
    for (size_t i = 0; i < h->dn_arc.size(); i++) {
        if (dn_tail) dn_tail[i] = h->dn_arc[i].x;
        if (dn_len) dn_len[i] = h->dn_arc[i].y;
    }
    for (size_t i = 0; i < h->up_arc.size(); i++) {
        if (up_head) up_head[i] = h->up_arc[i].x;
        if (up_len) up_len[i] = h->up_arc[i].y;
    }
    return PHAST_OK;
}

// ---------------------------------------------------------------- save / load
static const char MAGIC[8] = {'P', 'H', 'A', 'S', 'T', 'B', '2', '1'};

int phast_save(const phast_ctx* h, const char* path) {
    if (!h || !path) return PHAST_EINVAL;
    FILE* f = std::fopen(path, "wb");
    if (!f) return PHAST_EIO;
    uint64_t hdr[8] = {h->n, h->levels, h->m, h->shortcuts, h->rounds, h->dn_arc.size(), h->up_arc.size(), 0};
    bool ok = std::fwrite(MAGIC, 1, 8, f) == 8 && std::fwrite(hdr, 8, 8, f) == 8 &&
              std::fwrite(&h->build_seconds, 8, 1, f) == 1 &&
              std::fwrite(h->perm.data(), 4, h->n, f) == h->n &&
              std::fwrite(h->lvl_off.data(), 4, h->lvl_off.size(), f) == h->lvl_off.size() &&
              std::fwrite(h->dn_first.data(), 4, h->dn_first.size(), f) == h->dn_first.size() &&
              std::fwrite(h->up_first.data(), 4, h->up_first.size(), f) == h->up_first.size() &&
              std::fwrite(h->dn_arc.data(), 8, h->dn_arc.size(), f) == h->dn_arc.size() &&
              std::fwrite(h->up_arc.data(), 8, h->up_arc.size(), f) == h->up_arc.size();
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
    uint64_t hdr[8];
    bool ok = h && std::fread(magic, 1, 8, f) == 8 && std::memcmp(magic, MAGIC, 8) == 0 &&
              std::fread(hdr, 8, 8, f) == 8 && std::fread(&h->build_seconds, 8, 1, f) == 1;
    if (ok) {
        try {
            h->n = (uint32_t)hdr[0]; h->levels = (uint32_t)hdr[1]; h->m = hdr[2];
            h->shortcuts = hdr[3]; h->rounds = (uint32_t)hdr[4];
            h->perm.resize(h->n); h->iperm.resize(h->n);
            h->lvl_off.resize((size_t)h->levels + 1);
            h->dn_first.resize((size_t)h->n + 1); h->up_first.resize((size_t)h->n + 1);
            h->dn_arc.resize(hdr[5]); h->up_arc.resize(hdr[6]);
        } catch (const std::bad_alloc&) {
            std::fclose(f);
            return PHAST_ENOMEM;
        }
        ok = std::fread(h->perm.data(), 4, h->n, f) == h->n &&
             std::fread(h->lvl_off.data(), 4, h->lvl_off.size(), f) == h->lvl_off.size() &&
             std::fread(h->dn_first.data(), 4, h->dn_first.size(), f) == h->dn_first.size() &&
             std::fread(h->up_first.data(), 4, h->up_first.size(), f) == h->up_first.size() &&
             std::fread(h->dn_arc.data(), 8, h->dn_arc.size(), f) == h->dn_arc.size() &&
             std::fread(h->up_arc.data(), 8, h->up_arc.size(), f) == h->up_arc.size();
    }
    std::fclose(f);
    if (!ok) return PHAST_EIO;
    for (uint32_t v = 0; v < h->n; v++) {
        if (h->perm[v] >= h->n) return PHAST_EIO;
        h->iperm[h->perm[v]] = v;
    }
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
            cudaEventElapsedTime(&y, h->ev[i + 1], h->ev[i + 2]) != cudaSuccess) { cudaGetLastError(); return PHAST_ECUDA; }
        a += x; b += y;
    }
    *ms_up = a; *ms_sweep = b; *batches = h->ev_used / 3;
    return PHAST_OK;
}

uint64_t phast_launch_count(void) { return launches(); }

}  // extern "C"
