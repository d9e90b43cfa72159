// layout.cpp -- renumbering for the sweep.
//
// PHAST only needs the sweep to visit vertices in a reverse topological order of
// G-down: "(For correctness, any reverse topological order will do.)" (PAPER.md:14
// §III).  The paper picks level order with DFS order inside a level, "We assign lower
// IDs to vertices at higher levels; within each level, we keep the DFS order"
// (§IV-A), so that the sweep is "a simple linear sweep in increasing
// order of IDs".  LAYOUT_LEVELS reproduces that.
//
// LAYOUT_LEVELS_BFS keeps the level order but sorts each level by BFS
// rank of the input graph (a spatial sweep line), every other level reversed
// ("serpentine"), so that a level starts where the level above ended and the tail
// rows it reads first are still in L2 (profiles/r1_l2sim.md).
//
// LAYOUT_LEVELS_BANDS (the default) is LEVELS_BFS where the bottom levels are cut into
// BANDS of consecutive levels whose G-down arcs (both ends inside the band) form small
// connected components (C3: levels 0-4 hold 16.3 M vertices in components of at most
// 419).  Components are packed in BFS-rank order into groups; within each band level
// the vertices are sorted by group, so every group is a contiguous id range per level
// and can be swept by one CTA from the top of the band to its bottom without waiting
// for any other CTA: the rows a group writes are read back by the same group while they
// are still in L2 (profiles/r2_groupsim.md).  Still a reverse topological order:
// "(For correctness, any reverse topological order will do.)" (§III).
#include "layout.h"

#include <algorithm>
#include <numeric>

namespace phast {
namespace {

constexpr int kEinval = -1, kErange = -4, kEinternal = -7;

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


// union-find with path halving and union by size
struct UnionFind {
    std::vector<uint32_t> p, sz;
    explicit UnionFind(uint32_t n) : p(n), sz(n, 1) {}
    void reset(uint32_t v) { p[v] = v; sz[v] = 1; }
    uint32_t find(uint32_t x) {
        while (p[x] != x) { p[x] = p[p[x]]; x = p[x]; }
        return x;
    }
    uint32_t unite(uint32_t a, uint32_t b) {   // returns the size of the merged set
        a = find(a); b = find(b);
        if (a == b) return sz[a];
        if (sz[a] < sz[b]) std::swap(a, b);
        p[b] = a;
        sz[a] += sz[b];
        return sz[a];
    }
};

// Bands of LAYOUT_LEVELS_BANDS over CH levels (original ids).  Greedy from level 0
// up: a band [lo, hi) grows while the largest component of its internal G-down arcs
// has at most min(BAND_COMP_CAP, vertices / BAND_COMP_DIV) vertices and it has at most
// BAND_MAX_LEVELS levels; banding stops at the first band of one level.
// grp[v] = group of v inside its band (INF outside bands); returns the level ranges.
std::vector<std::pair<uint32_t, uint32_t>> make_bands(const ChResult& R, uint32_t levels,
                                                      const std::vector<uint32_t>& rank,
                                                      std::vector<uint32_t>& grp) {
    const uint32_t n = R.n;
    std::vector<std::pair<uint32_t, uint32_t>> out;
    grp.assign(n, 0xFFFFFFFFu);
    if (levels < 2) return out;
    // vertices by level, and G-down out-arcs by tail (the transpose of R.dn_*)
    std::vector<uint32_t> lf(levels + 1, 0), lv(n);
    for (uint32_t v = 0; v < n; v++) lf[R.level[v] + 1]++;
    for (uint32_t l = 0; l < levels; l++) lf[l + 1] += lf[l];
    {
        std::vector<uint32_t> fill(lf.begin(), lf.end() - 1);
        for (uint32_t v = 0; v < n; v++) lv[fill[R.level[v]]++] = v;
    }
    const uint64_t mdn = R.dn_first[n];
    std::vector<uint64_t> of((size_t)n + 1, 0);
    for (uint64_t e = 0; e < mdn; e++) of[R.dn_tail[e] + 1]++;
    for (uint32_t v = 0; v < n; v++) of[v + 1] += of[v];
    std::vector<uint32_t> oh(mdn);
    {
        std::vector<uint64_t> fill(of.begin(), of.end() - 1);
        for (uint32_t v = 0; v < n; v++)
            for (uint64_t e = R.dn_first[v]; e < R.dn_first[v + 1]; e++) oh[fill[R.dn_tail[e]]++] = v;
    }
    UnionFind uf(n);
    auto add_level = [&](uint32_t l, uint32_t lo) {   // level l joins the band [lo, l)
        uint32_t mx = 1;
        for (uint32_t i = lf[l]; i < lf[l + 1]; i++) uf.reset(lv[i]);
        if (l == lo) return mx;
        for (uint32_t i = lf[l]; i < lf[l + 1]; i++) {
            const uint32_t t = lv[i];
            for (uint64_t e = of[t]; e < of[t + 1]; e++)
                if (R.level[oh[e]] >= lo) mx = std::max(mx, uf.unite(t, oh[e]));
        }
        return mx;
    };
    uint32_t lo = 0;
    while (lo + 1 < levels) {
        uint32_t mx = add_level(lo, lo), hi = lo + 1;
        uint64_t nv = lf[lo + 1] - lf[lo];
        while (hi < levels && hi - lo < BAND_MAX_LEVELS) {
            mx = std::max(mx, add_level(hi, lo));
            nv += lf[hi + 1] - lf[hi];
            if (mx > BAND_COMP_CAP || (uint64_t)mx * BAND_COMP_DIV > nv) break;
            hi++;
        }
        if (hi - lo < 2) break;
        out.emplace_back(lo, hi);
        lo = hi;
    }
    // groups: components of each band (fresh union-find), ordered by their smallest BFS
    // rank, packed into groups of at least BAND_GROUP_MIN vertices
    for (const auto& b : out) {
        for (uint32_t l = b.first; l < b.second; l++) add_level(l, b.first);
        std::vector<std::pair<uint32_t, uint32_t>> comps;   // (smallest rank, root)
        for (uint32_t i = lf[b.first]; i < lf[b.second]; i++) {
            const uint32_t v = lv[i], r = uf.find(v);
            if (grp[r] == 0xFFFFFFFFu) { grp[r] = (uint32_t)comps.size(); comps.emplace_back(rank[v], r); }
            auto& c = comps[grp[r]];
            c.first = std::min(c.first, rank[v]);
        }
        for (const auto& c : comps) grp[c.second] = 0xFFFFFFFFu;
        std::sort(comps.begin(), comps.end());
        uint32_t g = 0, acc = 0;
        for (const auto& c : comps) {   // grp[root] = its group (roots are band vertices)
            grp[c.second] = g;
            acc += uf.sz[c.second];
            if (acc >= BAND_GROUP_MIN) { g++; acc = 0; }
        }
        std::vector<uint32_t> tmp(lf[b.second] - lf[b.first]);
        for (uint32_t i = lf[b.first]; i < lf[b.second]; i++) tmp[i - lf[b.first]] = grp[uf.find(lv[i])];
        for (uint32_t i = lf[b.first]; i < lf[b.second]; i++) grp[lv[i]] = tmp[i - lf[b.first]];
    }
    return out;
}

}  // namespace

int layout_build(const ChResult& R, const uint64_t* first, const uint32_t* head, uint32_t mode, Layout& L) {
    const uint32_t n = R.n;
    L.mode = mode;
    uint32_t levels = 0;
    for (uint32_t v = 0; v < n; v++) levels = std::max(levels, R.level[v] + 1);
    L.levels = levels;
    uint64_t mdn = R.dn_first[n], mup = R.up_first[n];
    if (mdn >= 0xFFFFFFFEull || mup >= 0xFFFFFFFEull) return kErange;

    std::vector<uint32_t> order(n);   // order[i] = original id with internal id i
    L.bands.clear();
    if (mode == LAYOUT_LEVELS || mode == LAYOUT_LEVELS_BFS || mode == LAYOUT_LEVELS_BANDS) {
        std::vector<uint32_t> cnt(levels, 0);
        for (uint32_t v = 0; v < n; v++) cnt[R.level[v]]++;
        L.lvl_off.assign(levels + 1, 0);
        for (uint32_t j = 0; j < levels; j++) L.lvl_off[j + 1] = L.lvl_off[j] + cnt[levels - 1 - j];
        std::vector<uint32_t> pos(levels);
        for (uint32_t j = 0; j < levels; j++) pos[levels - 1 - j] = L.lvl_off[j];
        std::vector<uint32_t> by(n);                 // within-level order: input id, or BFS rank
        std::iota(by.begin(), by.end(), 0u);
        std::vector<uint32_t> rank, grp;
        std::vector<std::pair<uint32_t, uint32_t>> bl;   // band level ranges [lo, hi), bottom first
        if (mode != LAYOUT_LEVELS) {
            rank = bfs_rank(n, first, head);
            std::sort(by.begin(), by.end(), [&](uint32_t a, uint32_t b) { return rank[a] < rank[b]; });
            if (mode == LAYOUT_LEVELS_BANDS) bl = make_bands(R, levels, rank, grp);
        }
        const uint32_t band_top = bl.empty() ? 0u : bl.back().second;   // CH levels [0, band_top) are banded
        if (!bl.empty()) {   // band levels: by group, then BFS rank (stable: by is in rank order)
            std::stable_sort(by.begin(), by.end(), [&](uint32_t a, uint32_t b) {
                const uint32_t ga = R.level[a] < band_top ? grp[a] : 0u, gb = R.level[b] < band_top ? grp[b] : 0u;
                return ga < gb;
            });
        }
        for (uint32_t v : by) order[pos[R.level[v]]++] = v;
        if (mode != LAYOUT_LEVELS)   // serpentine: odd levels in descending BFS rank, so a level starts
            for (uint32_t j = 0; j < levels; j++)   // where the level above ended (its rows still in L2):
                if (((levels - 1 - j) & 1u) && levels - 1 - j >= band_top)   // 7.8 % fewer tail-row misses
                    std::reverse(order.begin() + L.lvl_off[j], order.begin() + L.lvl_off[j + 1]);   // (r1_l2sim.md)
        for (size_t b = bl.size(); b-- > 0;) {   // bands top-most first; goff from the group counts
            Band B;
            B.seg_lo = levels - bl[b].second;
            B.seg_hi = levels - bl[b].first;
            uint32_t ng = 0;
            for (uint32_t j = B.seg_lo; j < B.seg_hi; j++)
                for (uint32_t r = L.lvl_off[j]; r < L.lvl_off[j + 1]; r++) ng = std::max(ng, grp[order[r]] + 1);
            B.ngroups = ng;
            B.goff.assign((size_t)(B.seg_hi - B.seg_lo) * (ng + 1), 0);
            for (uint32_t j = B.seg_lo; j < B.seg_hi; j++) {
                uint32_t* go = B.goff.data() + (size_t)(j - B.seg_lo) * (ng + 1);
                for (uint32_t r = L.lvl_off[j]; r < L.lvl_off[j + 1]; r++) go[grp[order[r]] + 1]++;
                go[0] = L.lvl_off[j];
                for (uint32_t g = 0; g < ng; g++) go[g + 1] += go[g];
            }
            L.bands.push_back(std::move(B));
        }
    } else {
        return kEinval;
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
    if (ok && check_bands(L) != 0) ok = false;
    return ok ? 0 : kEinternal;
}

int check_bands(const Layout& L) {
    const uint32_t nseg = L.lvl_off.empty() ? 0u : (uint32_t)L.lvl_off.size() - 1;
    uint32_t prev_lo = nseg;   // bands tile a suffix of the segments, top-most first, bottom band last
    for (size_t b = L.bands.size(); b-- > 0;) {
        const Band& B = L.bands[b];
        if (B.seg_hi != prev_lo || B.seg_lo + 2 > B.seg_hi || B.seg_hi - B.seg_lo > BAND_MAX_LEVELS || B.ngroups == 0 ||
            B.goff.size() != (size_t)(B.seg_hi - B.seg_lo) * (B.ngroups + 1))
            return kEinternal;
        prev_lo = B.seg_lo;
        const uint32_t base = L.lvl_off[B.seg_lo], end = L.lvl_off[B.seg_hi];
        std::vector<uint32_t> g_of(end - base);
        for (uint32_t j = B.seg_lo; j < B.seg_hi; j++) {
            const uint32_t* go = B.goff.data() + (size_t)(j - B.seg_lo) * (B.ngroups + 1);
            if (go[0] != L.lvl_off[j] || go[B.ngroups] != L.lvl_off[j + 1]) return kEinternal;
            for (uint32_t g = 0; g < B.ngroups; g++) {
                if (go[g] > go[g + 1]) return kEinternal;
                for (uint32_t r = go[g]; r < go[g + 1]; r++) g_of[r - base] = g;
            }
        }
        for (uint32_t r = base; r < end; r++)   // closed groups: every in-band tail in the head's group
            for (uint32_t e = L.dn_first[r]; e < L.dn_first[r + 1]; e++) {
                const uint32_t t = L.dn_arc[e].x;
                if (t >= base && g_of[t - base] != g_of[r - base]) return kEinternal;
            }
    }
    return 0;
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

}  // namespace phast
