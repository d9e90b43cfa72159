/*
 * phastgen/gen.c -- seeded synthetic inputs shared by the oracle side (tests/,
 * bench.py cpu_baseline) and the CUDA side (bench.py, tests/).  This module
 * holds NONE of the method's arithmetic: it only draws graphs and sources.
 *
 * Workloads follow the paper's benchmark instances in shape only:
 *   - Europe: "18 million vertices and 42 million arcs" (§II-A),
 *   - USA:    "24 million vertices and 58.3 million arcs" (§VIII-G),
 *   - travel-time lengths: "The length of each arc represents the travel time
 *     between its endpoints" (§VIII-A),
 *   - DFS layout: "IDs given by the order vertices are discovered during a DFS
 *     from a random vertex" (§VIII-B).
 * The recipe (lattice + road classes + shape points + DFS relabel) is stated in
 * DESIGN.md §"Input recipe".
 *
 * Output format: CSR of OUT-arcs, first[n+1] (uint64), head[m], len[m] (uint32),
 * the paper's first/arclist layout (§IV-A "first[v] denotes the
 * position in arclist of the first outgoing arc from v").
 *
 * Randomness: a counter-based generator (splitmix64 of seed ^ stream ^ index), so
 * every draw is a pure function of (seed, stream, index).
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

typedef struct {
    uint32_t n;
    uint64_t m;
    uint64_t *first;
    uint32_t *head;
    uint32_t *len;
} pg_graph;

static inline uint64_t mix64(uint64_t z) {
    z += 0x9E3779B97F4A7C15ull;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}
/* uniform 64-bit word for (seed, stream, index) */
static inline uint64_t rnd(uint64_t seed, uint64_t stream, uint64_t idx) {
    return mix64(mix64(seed ^ (stream * 0xD1B54A32D192ED03ull)) ^ idx);
}
/* uniform double in [0,1) */
static inline double rndu(uint64_t seed, uint64_t stream, uint64_t idx) {
    return (double)(rnd(seed, stream, idx) >> 11) * (1.0 / 9007199254740992.0);
}

void pg_free(pg_graph *g) {
    if (!g) return;
    free(g->first); free(g->head); free(g->len);
    g->first = NULL; g->head = NULL; g->len = NULL;
}

/* ------------------------------------------------------------------------- */
/* Exact W x H 4-neighbour grid, row-major ids v = W*y + x, every lattice edge in
 * both directions, each ARC with an independent length uniform in [lo, hi).
 * (BASELINE.json configs[0]: "100x100 synthetic road-like grid (10k vertices,
 * ~40k arcs, random uint32 lengths)").  Out-arcs of v are emitted in the order
 * -x, +x, -y, +y.  Returns 0 on success. */
int pg_grid(uint32_t W, uint32_t H, uint32_t lo, uint32_t hi, uint64_t seed, pg_graph *g) {
    memset(g, 0, sizeof(*g));
    if (W == 0 || H == 0 || hi <= lo) return -1;
    uint64_t n = (uint64_t)W * H;
    if (n > 0xFFFFFFFEull) return -1;
    uint64_t m = 2ull * ((uint64_t)(W - 1) * H + (uint64_t)W * (H - 1));
    g->n = (uint32_t)n; g->m = m;
    g->first = (uint64_t *)malloc((n + 1) * sizeof(uint64_t));
    g->head = (uint32_t *)malloc((m ? m : 1) * sizeof(uint32_t));
    g->len = (uint32_t *)malloc((m ? m : 1) * sizeof(uint32_t));
    if (!g->first || !g->head || !g->len) { pg_free(g); return -2; }
    uint64_t e = 0;
    uint64_t span = (uint64_t)hi - lo;
    for (uint32_t y = 0; y < H; y++)
        for (uint32_t x = 0; x < W; x++) {
            uint64_t v = (uint64_t)y * W + x;
            g->first[v] = e;
            int64_t nb[4] = {x > 0 ? (int64_t)v - 1 : -1, x + 1 < W ? (int64_t)v + 1 : -1,
                             y > 0 ? (int64_t)v - W : -1, y + 1 < H ? (int64_t)(v + W) : -1};
            for (int d = 0; d < 4; d++) {
                if (nb[d] < 0) continue;
                g->head[e] = (uint32_t)nb[d];
                g->len[e] = lo + (uint32_t)(rnd(seed, 1, e) % span);
                e++;
            }
        }
    g->first[n] = e;
    return e == m ? 0 : -3;
}

/* ------------------------------------------------------------------------- */
/* Road-like generator.
 *   lattice W x H of intersections; lattice edge on row/column i has road class
 *   c(i) = 3 if i%512==0 (motorway, speed 8), 2 if i%64==0 (highway, 4),
 *          1 if i%8==0 (arterial, 2), else 0 (local street, 1).
 *   class>=1 edges always kept; class-0 edges kept with probability p_keep; then
 *   dropped edges are re-added (Kruskal over a seeded random permutation) until the
 *   lattice is connected.  A spanning forest of the kept edges is fixed; non-tree
 *   class-0 edges become one-way (random direction) with probability oneway.
 *   Each kept edge is subdivided by s shape vertices, P(s=j) = shape_p[j], j<4.
 *   Edge travel time T = round(base * U(0.8,1.2) / speed), split over the s+1
 *   segments with weights U(0.5,1.5), every segment >= 1.  metric = 1 (travel
 *   DISTANCE, §VIII-G "generating upwards and downwards graphs with 410
 *   levels"): every class has speed 1, so the length is the geometric length.
 *   Finally ids are relabelled in DFS discovery order from a seeded random vertex
 *   (undirected DFS, neighbours in stored order).
 */
typedef struct { uint32_t a, b; uint8_t cls, keep, oneway, dir; } pg_edge;

static uint32_t uf_find(uint32_t *p, uint32_t x) {
    while (p[x] != x) { p[x] = p[p[x]]; x = p[x]; }
    return x;
}

static int road_class(uint32_t i) {
    if (i % 512 == 0) return 3;
    if (i % 64 == 0) return 2;
    if (i % 8 == 0) return 1;
    return 0;
}

int pg_road(uint32_t W, uint32_t H, double p_keep, const double *shape_p, double oneway,
            uint32_t base, uint64_t seed, uint32_t metric, pg_graph *g) {
    memset(g, 0, sizeof(*g));
    if (W < 2 || H < 2) return -1;
    uint64_t NI = (uint64_t)W * H;
    uint64_t NE = (uint64_t)(W - 1) * H + (uint64_t)W * (H - 1);
    pg_edge *E = (pg_edge *)malloc(NE * sizeof(pg_edge));
    uint32_t *uf = (uint32_t *)malloc(NI * sizeof(uint32_t));
    if (!E || !uf) { free(E); free(uf); return -2; }
    uint64_t k = 0;
    for (uint32_t y = 0; y < H; y++)
        for (uint32_t x = 0; x + 1 < W; x++) {
            pg_edge *e = &E[k++];
            e->a = y * W + x; e->b = y * W + x + 1; e->cls = (uint8_t)road_class(y);
        }
    for (uint32_t y = 0; y + 1 < H; y++)
        for (uint32_t x = 0; x < W; x++) {
            pg_edge *e = &E[k++];
            e->a = y * W + x; e->b = (y + 1) * W + x; e->cls = (uint8_t)road_class(x);
        }
    for (uint64_t i = 0; i < NE; i++) {
        pg_edge *e = &E[i];
        e->keep = e->cls >= 1 || rndu(seed, 2, i) < p_keep;
        e->oneway = 0; e->dir = 0;
    }
    /* spanning forest over kept edges, then connect with dropped edges in random order */
    for (uint64_t v = 0; v < NI; v++) uf[v] = (uint32_t)v;
    uint8_t *tree = (uint8_t *)calloc(NE, 1);
    uint64_t *perm = (uint64_t *)malloc(NE * sizeof(uint64_t));
    if (!tree || !perm) { free(E); free(uf); free(tree); free(perm); return -2; }
    for (uint64_t i = 0; i < NE; i++) {
        if (!E[i].keep) continue;
        uint32_t ra = uf_find(uf, E[i].a), rb = uf_find(uf, E[i].b);
        if (ra != rb) { uf[ra] = rb; tree[i] = 1; }
    }
    for (uint64_t i = 0; i < NE; i++) perm[i] = i;
    for (uint64_t i = NE; i > 1; i--) {           /* Fisher-Yates */
        uint64_t j = rnd(seed, 3, i) % i;
        uint64_t t = perm[i - 1]; perm[i - 1] = perm[j]; perm[j] = t;
    }
    for (uint64_t t = 0; t < NE; t++) {
        uint64_t i = perm[t];
        if (E[i].keep) continue;
        uint32_t ra = uf_find(uf, E[i].a), rb = uf_find(uf, E[i].b);
        if (ra != rb) { uf[ra] = rb; tree[i] = 1; E[i].keep = 1; }
    }
    free(perm);
    for (uint64_t i = 0; i < NE; i++)
        if (E[i].keep && !tree[i] && E[i].cls == 0 && rndu(seed, 4, i) < oneway) {
            E[i].oneway = 1; E[i].dir = (uint8_t)(rnd(seed, 5, i) & 1);
        }
    free(tree);
    free(uf);

    /* count vertices and arcs */
    double cum[4]; double acc = 0;
    for (int j = 0; j < 4; j++) { acc += shape_p[j]; cum[j] = acc; }
    uint8_t *ns = (uint8_t *)malloc(NE);
    uint64_t nv = NI, narcs = 0;
    for (uint64_t i = 0; i < NE; i++) {
        if (!E[i].keep) { ns[i] = 0; continue; }
        double u = rndu(seed, 6, i) * acc;
        int s = 0; while (s < 3 && u >= cum[s]) s++;
        ns[i] = (uint8_t)s;
        nv += s;
        narcs += (uint64_t)(s + 1) * (E[i].oneway ? 1 : 2);
    }
    if (nv > 0xFFFFFFFEull) { free(E); free(ns); return -1; }
    /* build arc list (tail, head, len) in generation order */
    uint32_t *at = (uint32_t *)malloc(narcs * sizeof(uint32_t));
    uint32_t *ah = (uint32_t *)malloc(narcs * sizeof(uint32_t));
    uint32_t *al = (uint32_t *)malloc(narcs * sizeof(uint32_t));
    if (!at || !ah || !al || !ns) { free(E); free(ns); free(at); free(ah); free(al); return -2; }
    uint64_t na = 0; uint32_t next_v = (uint32_t)NI;
    static const double speed[4] = {1.0, 2.0, 4.0, 8.0};
    for (uint64_t i = 0; i < NE; i++) {
        if (!E[i].keep) continue;
        int s = ns[i];
        double T = (double)base * (0.8 + 0.4 * rndu(seed, 7, i)) / (metric ? 1.0 : speed[E[i].cls]);
        double w[4], ws = 0;
        for (int j = 0; j <= s; j++) { w[j] = 0.5 + rndu(seed, 8, i * 4 + j); ws += w[j]; }
        uint32_t chain[5];
        chain[0] = E[i].a;
        for (int j = 1; j <= s; j++) chain[j] = next_v++;
        chain[s + 1] = E[i].b;
        for (int j = 0; j <= s; j++) {
            double L = T * w[j] / ws;
            uint32_t l = (uint32_t)(L + 0.5);
            if (l < 1) l = 1;
            uint32_t u = chain[j], v = chain[j + 1];
            if (!E[i].oneway || E[i].dir == 0) { at[na] = u; ah[na] = v; al[na] = l; na++; }
            if (!E[i].oneway || E[i].dir == 1) { at[na] = v; ah[na] = u; al[na] = l; na++; }
        }
    }
    free(E); free(ns);
    uint32_t n = (uint32_t)nv;
    /* undirected adjacency for the DFS */
    uint64_t *ufirst = (uint64_t *)calloc((uint64_t)n + 1, sizeof(uint64_t));
    uint32_t *uadj = (uint32_t *)malloc(2 * na * sizeof(uint32_t));
    if (!ufirst || !uadj) { free(at); free(ah); free(al); free(ufirst); free(uadj); return -2; }
    for (uint64_t e = 0; e < na; e++) { ufirst[at[e] + 1]++; ufirst[ah[e] + 1]++; }
    for (uint64_t v = 0; v < n; v++) ufirst[v + 1] += ufirst[v];
    uint64_t *fill = (uint64_t *)malloc((uint64_t)n * sizeof(uint64_t));
    memcpy(fill, ufirst, (uint64_t)n * sizeof(uint64_t));
    for (uint64_t e = 0; e < na; e++) { uadj[fill[at[e]]++] = ah[e]; uadj[fill[ah[e]]++] = at[e]; }
    /* iterative DFS from a seeded random vertex: newid[v] = discovery index */
    uint32_t *newid = (uint32_t *)malloc((uint64_t)n * sizeof(uint32_t));
    uint32_t *stk = (uint32_t *)malloc((uint64_t)n * sizeof(uint32_t));
    for (uint64_t v = 0; v < n; v++) newid[v] = 0xFFFFFFFFu;
    uint32_t cnt = 0;
    uint32_t start = (uint32_t)(rnd(seed, 9, 0) % n);
    for (uint64_t r = 0; r < n; r++) {
        uint32_t root = (uint32_t)((start + r) % n);
        if (newid[root] != 0xFFFFFFFFu) continue;
        uint64_t sp = 0;
        newid[root] = cnt++; stk[sp++] = root;
        /* fill[v] reused as the per-vertex neighbour cursor */
        while (sp) {
            uint32_t v = stk[sp - 1];
            if (fill[v] == ufirst[v + 1]) { sp--; continue; }
            uint32_t w = uadj[fill[v]++];
            if (newid[w] == 0xFFFFFFFFu) { newid[w] = cnt++; stk[sp++] = w; }
        }
    }
    /* reset cursors (fill was advanced to ufirst[v+1]) -- not needed further */
    free(stk); free(uadj); free(ufirst);
    /* emit CSR in new ids, arcs of a tail in generation order */
    g->n = n; g->m = na;
    g->first = (uint64_t *)calloc((uint64_t)n + 1, sizeof(uint64_t));
    g->head = (uint32_t *)malloc(na * sizeof(uint32_t));
    g->len = (uint32_t *)malloc(na * sizeof(uint32_t));
    if (!g->first || !g->head || !g->len) { free(at); free(ah); free(al); free(newid); free(fill); pg_free(g); return -2; }
    for (uint64_t e = 0; e < na; e++) g->first[newid[at[e]] + 1]++;
    for (uint64_t v = 0; v < n; v++) g->first[v + 1] += g->first[v];
    for (uint64_t v = 0; v < n; v++) fill[v] = g->first[v];
    for (uint64_t e = 0; e < na; e++) {
        uint64_t p = fill[newid[at[e]]]++;
        g->head[p] = newid[ah[e]]; g->len[p] = al[e];
    }
    free(at); free(ah); free(al); free(newid); free(fill);
    return 0;
}

/* k distinct-or-not sources: uniform in [0,n), without replacement when
 * distinct != 0 (requires count <= n), via a seeded partial Fisher-Yates on a
 * hash map-free rejection scheme (count << n in every config). */
int pg_sources(uint32_t n, uint64_t count, int distinct, uint64_t seed, uint32_t *out) {
    if (n == 0) return -1;
    if (distinct && count > n) return -1;
    if (!distinct || count * 4 > n) {
        if (distinct) {                       /* dense: shuffle a full permutation prefix */
            uint32_t *p = (uint32_t *)malloc((uint64_t)n * sizeof(uint32_t));
            if (!p) return -2;
            for (uint64_t i = 0; i < n; i++) p[i] = (uint32_t)i;
            for (uint64_t i = 0; i < count; i++) {
                uint64_t j = i + rnd(seed, 10, i) % (n - i);
                uint32_t t = p[i]; p[i] = p[j]; p[j] = t;
                out[i] = p[i];
            }
            free(p);
        } else {
            for (uint64_t i = 0; i < count; i++) out[i] = (uint32_t)(rnd(seed, 10, i) % n);
        }
        return 0;
    }
    /* sparse distinct: rejection with a small open-addressing set */
    uint64_t cap = 16; while (cap < count * 4) cap <<= 1;
    uint32_t *set = (uint32_t *)malloc(cap * sizeof(uint32_t));
    if (!set) return -2;
    for (uint64_t i = 0; i < cap; i++) set[i] = 0xFFFFFFFFu;
    uint64_t got = 0, draw = 0;
    while (got < count) {
        uint32_t v = (uint32_t)(rnd(seed, 10, draw++) % n);
        uint64_t h = mix64(v) & (cap - 1);
        int dup = 0;
        while (set[h] != 0xFFFFFFFFu) { if (set[h] == v) { dup = 1; break; } h = (h + 1) & (cap - 1); }
        if (dup) continue;
        set[h] = v; out[got++] = v;
    }
    free(set);
    return 0;
}

/* Uniform random digraph for small oracle pins: n vertices, m arcs with tails and
 * heads uniform (self-loops and parallel arcs included), lengths uniform in
 * [lo, hi] (inclusive, 64-bit span so hi may be 0xFFFFFFFF).  CSR by tail. */
int pg_random_digraph(uint32_t n, uint64_t m, uint32_t lo, uint32_t hi, uint64_t seed, pg_graph *g) {
    memset(g, 0, sizeof(*g));
    if (n == 0 || hi < lo) return -1;
    g->n = n; g->m = m;
    g->first = (uint64_t *)calloc((uint64_t)n + 1, sizeof(uint64_t));
    g->head = (uint32_t *)malloc((m ? m : 1) * sizeof(uint32_t));
    g->len = (uint32_t *)malloc((m ? m : 1) * sizeof(uint32_t));
    uint32_t *tail = (uint32_t *)malloc((m ? m : 1) * sizeof(uint32_t));
    uint64_t *fill = (uint64_t *)malloc((uint64_t)n * sizeof(uint64_t));
    if (!g->first || !g->head || !g->len || !tail || !fill) { free(tail); free(fill); pg_free(g); return -2; }
    uint64_t span = (uint64_t)hi - lo + 1;
    for (uint64_t e = 0; e < m; e++) { tail[e] = (uint32_t)(rnd(seed, 11, e) % n); g->first[tail[e] + 1]++; }
    for (uint64_t v = 0; v < n; v++) g->first[v + 1] += g->first[v];
    for (uint64_t v = 0; v < n; v++) fill[v] = g->first[v];
    for (uint64_t e = 0; e < m; e++) {
        uint64_t p = fill[tail[e]]++;
        g->head[p] = (uint32_t)(rnd(seed, 12, e) % n);
        g->len[p] = (uint32_t)(lo + rnd(seed, 13, e) % span);
    }
    free(tail); free(fill);
    return 0;
}
