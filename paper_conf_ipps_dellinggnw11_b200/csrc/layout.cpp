// layout.cpp -- renumbering for the sweep.
//
// PHAST only needs the sweep to visit vertices in a reverse topological order of
// G-down: "(For correctness, any reverse topological order will do.)" (PAPER.md:14
// §III).  The paper picks level order with DFS order inside a level, "We assign lower
// IDs to vertices at higher levels; within each level, we keep the DFS order"
// (§IV-A), so that the sweep is "a simple linear sweep in increasing
// order of IDs".  LAYOUT_LEVELS reproduces that.
//
// LAYOUT_DIAGONAL keeps the paper's level order for the few vertices of the top
// levels (>= cut) and interleaves the bottom levels -- which hold almost all
// vertices and whose G-down arcs are short (level-0 in-arcs are original arcs) -- in
// "diagonals": with band(v) = rank(v) / delta (BFS rank, below) and per-level offsets
// o(l), key(v) = band(v) + o(L(v)); o is the smallest non-negative offset with
// key(tail) < key(head) on every bottom arc, computed top-down by level.  Diagonal j
// holds the bottom vertices with key j, so a diagonal never holds both ends of an arc,
// and each diagonal touches only a few consecutive bands of every bottom level: a
// tail row is written shortly before its bottom-level heads read it and stays in L2,
// where a level-by-level pass re-reads it from HBM once per level of its heads
// (profiles/r1_l2sim.md).
//
// LAYOUT_WAVEFRONT keeps the linear sweep but chooses a
// different topological order, one that keeps label rows in the B200's L2 cache.
//   rank(v) = BFS discovery order of the input graph (undirected) from a
//             pseudo-peripheral vertex: a spatial sweep line across the network.
//   key(v)  = min(rank(v), min over G-down arcs (v, w) of key(w) - delta),
//             computed bottom-up by CH level.
//   Internal ids sort vertices by (key, level descending, rank).
// Every G-down arc (u, w) has key(u) <= key(w) - delta < key(w), so the tail gets
// the smaller id and the order is topological.  A tail row is written about delta
// positions before the first head that reads it, and all its heads lie nearby on the
// same wavefront.  The row is therefore re-read from L2 instead of HBM, whereas
// level-by-level passes re-read it once per level of its heads.
#include "layout.h"

#include <algorithm>
#include <cstdlib>
#include <numeric>

namespace phast {
namespace {

constexpr int kErange = -4, kEinternal = -7;

// BFS discovery order over the undirected version of the input graph, restarted
// from the lowest unvisited id on disconnected inputs.  Returns rank[v].
std::vector<uint32_t> bfs_rank(uint32_t n, const uint64_t* first, const uint32_t* head) {
    uint64_t m = first[n];
    std::vector<uint64_t> uf((size_t)n + 1, 0);
    for (uint32_t u = 0; u < n; u++) {
        uf[u + 1] += first[u + 1] - first[u];
        for (uint64_t e = first[u]; e < first[u + 1]; e++) uf[head[e] + 1]++;
    }
    for (uint32_t v = 0; v < n; v++) uf[v + 1] += uf[v];
    std::vector<uint32_t> adj(2 * m);
    {
        std::vector<uint64_t> fill(uf.begin(), uf.end() - 1);
        for (uint32_t u = 0; u < n; u++)
            for (uint64_t e = first[u]; e < first[u + 1]; e++) {
                adj[fill[u]++] = head[e];
                adj[fill[head[e]]++] = u;
            }
    }
    std::vector<uint32_t> rank(n, 0xFFFFFFFFu), queue(n);
    auto bfs_all = [&](uint32_t start) {
        std::fill(rank.begin(), rank.end(), 0xFFFFFFFFu);
        uint32_t cnt = 0, qh = 0, qt = 0;
        uint32_t next_root = 0;
        uint32_t root = start;
        for (;;) {
            rank[root] = cnt++;
            queue[qt++] = root;
            while (qh < qt) {
                uint32_t u = queue[qh++];
                for (uint64_t e = uf[u]; e < uf[u + 1]; e++) {
                    uint32_t w = adj[e];
                    if (rank[w] == 0xFFFFFFFFu) { rank[w] = cnt++; queue[qt++] = w; }
                }
            }
            while (next_root < n && rank[next_root] != 0xFFFFFFFFu) next_root++;
            if (next_root >= n) break;
            root = next_root;
        }
        return queue[n - 1];   // last discovered vertex
    };
    uint32_t far = bfs_all(0);   // pseudo-peripheral start: the last vertex of a first BFS
    bfs_all(far);
    return rank;
}

}  // namespace

int layout_build(const ChResult& R, const uint64_t* first, const uint32_t* head, uint32_t mode, uint32_t delta,
                 Layout& L) {
    const uint32_t n = R.n;
    L.mode = mode;
    L.delta = delta;
    uint32_t levels = 0;
    for (uint32_t v = 0; v < n; v++) levels = std::max(levels, R.level[v] + 1);
    L.levels = levels;
    uint64_t mdn = R.dn_first[n], mup = R.up_first[n];
    if (mdn >= 0xFFFFFFFEull || mup >= 0xFFFFFFFEull) return kErange;

    std::vector<uint32_t> order(n);   // order[i] = original id with internal id i
    if (mode == LAYOUT_LEVELS || mode == LAYOUT_LEVELS_BFS) {
        std::vector<uint32_t> cnt(levels, 0);
        for (uint32_t v = 0; v < n; v++) cnt[R.level[v]]++;
        L.lvl_off.assign(levels + 1, 0);
        for (uint32_t j = 0; j < levels; j++) L.lvl_off[j + 1] = L.lvl_off[j] + cnt[levels - 1 - j];
        std::vector<uint32_t> pos(levels);
        for (uint32_t j = 0; j < levels; j++) pos[levels - 1 - j] = L.lvl_off[j];
        std::vector<uint32_t> by(n);                 // within-level order: input id, or BFS rank
        std::iota(by.begin(), by.end(), 0u);
        if (mode == LAYOUT_LEVELS_BFS) {
            std::vector<uint32_t> rank = bfs_rank(n, first, head);
            std::sort(by.begin(), by.end(), [&](uint32_t a, uint32_t b) { return rank[a] < rank[b]; });
        }
        for (uint32_t v : by) order[pos[R.level[v]]++] = v;
        if (mode == LAYOUT_LEVELS_BFS)   // serpentine: odd levels in descending BFS rank, so a
            for (uint32_t j = 0; j < levels; j++)   // level starts where the level above ended (its rows
                if ((levels - 1 - j) & 1u)          // still in L2): 7.8 % fewer tail-row misses (r1_l2sim.md)
                    std::reverse(order.begin() + L.lvl_off[j], order.begin() + L.lvl_off[j + 1]);
    } else if (mode == LAYOUT_DIAGONAL) {
        std::vector<uint32_t> rank = bfs_rank(n, first, head);
        std::vector<uint32_t> cnt(levels, 0);
        for (uint32_t v = 0; v < n; v++) cnt[R.level[v]]++;
        // cut: the lowest level whose part above holds at most n / 256 vertices
        uint32_t cut = levels;
        {
            uint64_t above = 0;
            while (cut > 1 && above + cnt[cut - 1] <= n / 256) above += cnt[--cut];
        }
        // experiment knobs: the cut level, and the lag (key(tail) <= key(head) - lag, so
        // that a persistent sweep may run diagonal j while diagonals > j - lag finish)
        if (const char* e = std::getenv("PHAST_DIAG_CUT")) cut = std::max(1u, std::min<uint32_t>(levels, std::atoi(e)));
        uint32_t lag = 1;
        if (const char* e = std::getenv("PHAST_DIAG_LAG")) lag = std::max(1, std::min(8, std::atoi(e)));
        L.cut = cut;
        L.lag = lag;
        const uint32_t band_w = std::max(1u, delta);
        auto band = [&](uint32_t v) { return (int64_t)(rank[v] / band_w); };
        std::vector<int64_t> o(levels, 0);
        {   // offsets top-down: o(l) = max over bottom arcs (t -> v), L(v) = l, of o(L(t)) + band(t) - band(v) + 1
            std::vector<std::vector<uint32_t>> by_level(cut);
            for (uint32_t v = 0; v < n; v++)
                if (R.level[v] < cut) by_level[R.level[v]].push_back(v);
            for (int64_t l = (int64_t)cut - 1; l >= 0; l--)
                for (uint32_t v : by_level[l])
                    for (uint64_t e = R.dn_first[v]; e < R.dn_first[v + 1]; e++) {
                        const uint32_t t = R.dn_tail[e];
                        if (R.level[t] < cut) o[l] = std::max(o[l], o[R.level[t]] + band(t) - band(v) + lag);
                    }
        }
        std::iota(order.begin(), order.end(), 0u);
        auto key = [&](uint32_t v) { return R.level[v] >= cut ? -1 - (int64_t)R.level[v] : band(v) + o[R.level[v]]; };
        std::sort(order.begin(), order.end(), [&](uint32_t a, uint32_t b) {
            const int64_t ka = key(a), kb = key(b);
            if (ka != kb) return ka < kb;
            if (R.level[a] != R.level[b]) return R.level[a] > R.level[b];
            return rank[a] < rank[b];
        });
        // one segment per top level, then one per bottom key VALUE, empty ones included:
        // key(head) - key(tail) >= lag must hold for segment indices too, so that a
        // lagged schedule (segment j waits for j - lag) sees every tail finished
        L.lvl_off.assign(1, 0);
        for (uint32_t r = 1; r <= n; r++) {
            if (r < n && key(order[r]) == key(order[r - 1])) continue;
            const int64_t kp = key(order[r - 1]);
            if (r < n && kp >= 0)
                for (int64_t kk = kp + 1; kk < key(order[r]); kk++) L.lvl_off.push_back(r);   // empty keys
            L.lvl_off.push_back(r);
        }
    } else {
        std::vector<uint32_t> rank = bfs_rank(n, first, head);
        std::vector<int64_t> key(n);
        for (uint32_t v = 0; v < n; v++) key[v] = rank[v];
        // G-down arcs (t -> v) bucketed by the level of their tail; heads are on lower
        // levels, so processing tail levels in ascending order sees final head keys.
        std::vector<uint64_t> lstart((size_t)levels + 1, 0);
        for (uint32_t v = 0; v < n; v++)
            for (uint64_t e = R.dn_first[v]; e < R.dn_first[v + 1]; e++) lstart[R.level[R.dn_tail[e]] + 1]++;
        for (uint32_t j = 0; j < levels; j++) lstart[j + 1] += lstart[j];
        std::vector<std::pair<uint32_t, uint32_t>> byl(mdn);   // (tail, head)
        {
            std::vector<uint64_t> fill(lstart.begin(), lstart.end() - 1);
            for (uint32_t v = 0; v < n; v++)
                for (uint64_t e = R.dn_first[v]; e < R.dn_first[v + 1]; e++) {
                    uint32_t t = R.dn_tail[e];
                    byl[fill[R.level[t]]++] = {t, v};
                }
        }
        for (uint32_t j = 0; j < levels; j++)
            for (uint64_t i = lstart[j]; i < lstart[j + 1]; i++) {
                const uint32_t t = byl[i].first, w = byl[i].second;
                key[t] = std::min(key[t], key[w] - (int64_t)delta);
            }
        std::iota(order.begin(), order.end(), 0u);
        std::sort(order.begin(), order.end(), [&](uint32_t a, uint32_t b) {
            if (key[a] != key[b]) return key[a] < key[b];
            if (R.level[a] != R.level[b]) return R.level[a] > R.level[b];
            return rank[a] < rank[b];
        });
    }
    L.perm.assign(n, 0);
    L.iperm = order;
    L.level.resize(n);
    for (uint32_t r = 0; r < n; r++) {
        L.perm[order[r]] = r;
        L.level[r] = R.level[order[r]];
    }
    L.dn_first.assign((size_t)n + 1, 0);
    L.up_first.assign((size_t)n + 1, 0);
    L.dn_arc.resize(mdn);
    L.up_arc.resize(mup);
    for (uint32_t r = 0; r < n; r++) {
        uint32_t v = L.iperm[r];
        L.dn_first[r + 1] = L.dn_first[r] + (uint32_t)(R.dn_first[v + 1] - R.dn_first[v]);
        L.up_first[r + 1] = L.up_first[r] + (uint32_t)(R.up_first[v + 1] - R.up_first[v]);
    }
    bool ok = true;
    auto by_x = [](const Arc& a, const Arc& b) { return a.x < b.x || (a.x == b.x && a.y < b.y); };
    for (uint32_t r = 0; r < n; r++) {
        uint32_t v = L.iperm[r];
        uint32_t p = L.dn_first[r];
        for (uint64_t e = R.dn_first[v]; e < R.dn_first[v + 1]; e++) {
            uint32_t t = R.dn_tail[e];
            // Lemma 4.1: (t, v) in A-down => L(t) > L(v) (§IV-A); and the tail's
            // row is final before the head is scanned: internal id of t < r
            if (!(R.level[t] > R.level[v]) || !(L.perm[t] < r)) ok = false;
            L.dn_arc[p++] = Arc{L.perm[t], R.dn_len[e]};
        }
        std::sort(L.dn_arc.begin() + L.dn_first[r], L.dn_arc.begin() + L.dn_first[r + 1], by_x);
        p = L.up_first[r];
        for (uint64_t e = R.up_first[v]; e < R.up_first[v + 1]; e++) {
            uint32_t w = R.up_head[e];
            if (!(R.level[w] > R.level[v])) ok = false;        // same rule for A-up
            L.up_arc[p++] = Arc{L.perm[w], R.up_len[e]};
        }
        std::sort(L.up_arc.begin() + L.up_first[r], L.up_arc.begin() + L.up_first[r + 1], by_x);
    }
    if (ok && !L.lvl_off.empty()) {   // segments: no G-down arc inside one segment
        std::vector<uint32_t> seg(n);
        for (uint32_t j = 0; j + 1 < L.lvl_off.size(); j++)
            for (uint32_t r = L.lvl_off[j]; r < L.lvl_off[j + 1]; r++) seg[r] = j;
        for (uint32_t r = 0; r < n && ok; r++)
            for (uint32_t e = L.dn_first[r]; e < L.dn_first[r + 1]; e++)
                if (!(seg[L.dn_arc[e].x] < seg[r])) { ok = false; break; }
    }
    return ok ? 0 : kEinternal;
}

int build_in_csr(Layout& L, uint32_t n, const uint64_t* first, const uint32_t* head, const uint32_t* len) {
    std::vector<uint64_t> cnt((size_t)n + 1, 0);
    for (uint32_t u = 0; u < n; u++)
        for (uint64_t e = first[u]; e < first[u + 1]; e++)
            if (head[e] != u && len[e] != 0xFFFFFFFFu) cnt[L.perm[head[e]] + 1]++;
    for (uint32_t r = 0; r < n; r++) cnt[r + 1] += cnt[r];
    if (cnt[n] >= 0xFFFFFFFEull) return kErange;
    L.in_first.assign(cnt.begin(), cnt.end());
    L.in_arc.resize(cnt[n]);
    std::vector<uint64_t> fill(cnt.begin(), cnt.end() - 1);
    for (uint32_t u = 0; u < n; u++)          // increasing input arc index
        for (uint64_t e = first[u]; e < first[u + 1]; e++)
            if (head[e] != u && len[e] != 0xFFFFFFFFu) L.in_arc[fill[L.perm[head[e]]]++] = Arc{L.perm[u], len[e]};
    return 0;
}

int plan_warp_chunks(const Layout& L, uint32_t cap, uint32_t workers, WarpPlan& P, uint32_t cap_arcs) {
    const uint32_t n = (uint32_t)L.perm.size();
    if (cap == 0 || workers == 0) return kEinternal;
    std::vector<uint32_t> cb{0}, chunk_of(n);
    uint32_t s = 0;
    for (uint32_t v = 0; v < n; v++) {
        bool cut = (v - s == cap);
        if (!cut && v > s && cap_arcs && L.dn_first[v + 1] - L.dn_first[s] > cap_arcs) cut = true;
        if (!cut && v > s)
            for (uint32_t e = L.dn_first[v]; e < L.dn_first[v + 1]; e++)
                if (L.dn_arc[e].x >= s) { cut = true; break; }
        if (cut) { cb.push_back(v); s = v; }
        chunk_of[v] = (uint32_t)cb.size() - 1;
    }
    cb.push_back(n);
    const uint32_t nch = (uint32_t)cb.size() - 1;
    P.meta.assign((size_t)nch * 4, 0);
    P.deps.clear();
    std::vector<uint32_t> tmp;
    for (uint32_t c = 0; c < nch; c++) {
        tmp.clear();
        bool prev = false;
        for (uint32_t e = L.dn_first[cb[c]]; e < L.dn_first[cb[c + 1]]; e++) {
            uint32_t x = chunk_of[L.dn_arc[e].x];
            if (x >= c) return kEinternal;                       // not topological
            if (x % workers != c % workers) tmp.push_back(x);     // same worker: already done
            else if (x + workers == c) prev = true;               // the worker's previous chunk
        }
        std::sort(tmp.begin(), tmp.end());
        tmp.erase(std::unique(tmp.begin(), tmp.end()), tmp.end());
        if (P.deps.size() + tmp.size() >= 0x7FFFFFF0ull) return kErange;
        P.meta[4 * (size_t)c + 0] = cb[c];
        P.meta[4 * (size_t)c + 1] = cb[c + 1];
        P.meta[4 * (size_t)c + 2] = (uint32_t)P.deps.size();
        P.deps.insert(P.deps.end(), tmp.begin(), tmp.end());
        P.meta[4 * (size_t)c + 3] = (uint32_t)P.deps.size() | (prev ? 0x80000000u : 0u);
    }
    P.chunks = nch;
    return 0;
}

int plan_chunks(const Layout& L, uint32_t cap, uint32_t grid, ChunkPlan& P, uint32_t cap_arcs, uint32_t lag,
                uint32_t limit) {
    const uint32_t n = limit ? limit : (uint32_t)L.perm.size();
    if (cap == 0 || grid == 0 || lag == 0) return kEinternal;
    // 1. chunk boundaries and each chunk's latest tail chunk (unpadded numbering)
    std::vector<uint32_t> cb{0}, chunk_of(n);
    uint32_t s = 0;
    for (uint32_t v = 0; v < n; v++) {
        bool cut = (v - s == cap);
        if (!cut && v > s && cap_arcs && L.dn_first[v + 1] - L.dn_first[s] > cap_arcs) cut = true;
        if (!cut && v > s)
            for (uint32_t e = L.dn_first[v]; e < L.dn_first[v + 1]; e++)
                if (L.dn_arc[e].x >= s) { cut = true; break; }
        if (cut) { cb.push_back(v); s = v; }
        chunk_of[v] = (uint32_t)cb.size() - 1;
    }
    cb.push_back(n);
    const uint32_t nch = (uint32_t)cb.size() - 1;
    // 2. slots with padding so that a dependency is always >= lag iterations earlier
    std::vector<uint32_t> slot(nch);
    P.slot_v.clear();
    P.dep.clear();
    uint64_t next = 0;
    P.pads = 0;
    for (uint32_t c = 0; c < nch; c++) {
        int64_t d = -1;
        for (uint32_t e = L.dn_first[cb[c]]; e < L.dn_first[cb[c + 1]]; e++)
            d = std::max<int64_t>(d, chunk_of[L.dn_arc[e].x]);
        if (d >= (int64_t)c) return kEinternal;
        uint64_t j = next;
        if (d >= 0 && slot[d] / grid + lag > j / grid) j = (uint64_t)(slot[d] / grid + lag) * grid;
        if (j > 0xFFFFFFF0ull) return kErange;
        for (uint64_t q = next; q < j; q++) {              // pads: empty ranges
            P.slot_v.push_back(cb[c]);
            P.dep.push_back(0);
            P.pads++;
        }
        slot[c] = (uint32_t)j;
        P.slot_v.push_back(cb[c]);
        P.dep.push_back(d < 0 ? 0u : slot[d] / grid + 1u);
        next = j + 1;
    }
    P.slot_v.push_back(n);
    P.chunks = nch;
    P.slots = (uint32_t)P.dep.size();
    return 0;
}

int plan_waves(const Layout& L, uint32_t cap, uint32_t cap_arcs, uint32_t T, uint32_t window, WavePlan& P) {
    const uint32_t n = (uint32_t)L.perm.size();
    if (cap == 0 || cap > 255 || T == 0) return kEinternal;
    // 1. chunk boundaries (no chunk holds both ends of a G-down arc)
    std::vector<uint32_t> cb{0}, chunk_of(n);
    uint32_t s = 0;
    for (uint32_t v = 0; v < n; v++) {
        bool cut = (v - s == cap);
        if (!cut && v > s && cap_arcs && L.dn_first[v + 1] - L.dn_first[s] > cap_arcs) cut = true;
        if (!cut && v > s)
            for (uint32_t e = L.dn_first[v]; e < L.dn_first[v + 1]; e++)
                if (L.dn_arc[e].x >= s) { cut = true; break; }
        if (cut) { cb.push_back(v); s = v; }
        chunk_of[v] = (uint32_t)cb.size() - 1;
    }
    cb.push_back(n);
    const uint32_t nch = (uint32_t)cb.size() - 1;
    // 2. first-fit placement in id order
    std::vector<uint32_t> wave(nch), dep(nch), fill, nxt;   // nxt[w]: a later wave to try when w is full
    auto grow = [&](uint32_t w) {
        while (fill.size() <= w) { nxt.push_back((uint32_t)fill.size()); fill.push_back(0); }
    };
    auto find = [&](uint32_t w) {   // first wave >= w with a free slot (path-compressed skips)
        grow(w);
        uint32_t r = w;
        while (fill[r] == T) { r = nxt[r]; grow(r); }
        while (w != r) { const uint32_t nx = nxt[w]; nxt[w] = r; w = nx; }
        return r;
    };
    uint32_t hi = 0;
    for (uint32_t c = 0; c < nch; c++) {
        int64_t dw = -1;
        for (uint32_t e = L.dn_first[cb[c]]; e < L.dn_first[cb[c + 1]]; e++) {
            const uint32_t x = chunk_of[L.dn_arc[e].x];
            if (x >= c) return kEinternal;                     // not topological
            dw = std::max<int64_t>(dw, wave[x]);
        }
        uint32_t lo = (uint32_t)(dw + 1);
        if (hi > window) lo = std::max(lo, hi - window);
        const uint32_t w = find(lo);
        if (w > 0xFFFFF0u) return kErange;
        wave[c] = w;
        dep[c] = (uint32_t)(dw + 1);
        if (++fill[w] == T) nxt[w] = w + 1;
        hi = std::max(hi, w);
        const uint64_t lag = dw < 0 ? 4 : w - (uint64_t)dw;
        P.lag_hist[std::min<uint64_t>(lag, 4) - 1]++;
    }
    // 3. slot table
    const uint32_t waves = nch ? hi + 1 : 0;
    P.desc.assign((size_t)4 * waves * T, 0);
    std::fill(fill.begin(), fill.end(), 0);
    for (uint32_t c = 0; c < nch; c++) {
        const size_t sl = (size_t)wave[c] * T + fill[wave[c]]++;
        uint32_t* q = &P.desc[4 * sl];
        q[0] = cb[c];
        q[1] = (cb[c + 1] - cb[c]) | (dep[c] << 8);
        q[2] = L.dn_first[cb[c]];
        q[3] = L.dn_first[cb[c + 1]];
    }
    P.chunks = nch;
    P.waves = waves;
    P.pads = (uint32_t)((uint64_t)waves * T - nch);
    return 0;
}

}  // namespace phast
