// layout.cpp -- renumbering for the sweep.
//
// PHAST only needs the sweep to visit vertices in a reverse topological order of
// G-down: "(For correctness, any reverse topological order will do.)" (PAPER.md:14
// §III).  The paper picks level order with DFS order inside a level, "We assign lower
// IDs to vertices at higher levels; within each level, we keep the DFS order"
// (§IV-A), so that the sweep is "a simple linear sweep in increasing
// order of IDs".  LAYOUT_LEVELS reproduces that.
//
// LAYOUT_LEVELS_BFS (the default) keeps the level order but sorts each level by BFS
// rank of the input graph (a spatial sweep line), every other level reversed
// ("serpentine"), so that a level starts where the level above ended and the tail
// rows it reads first are still in L2 (profiles/r1_l2sim.md).
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

}  // namespace phast
