// layout.h -- vertex renumbering and the G-up / G-down CSRs in internal ids.
// Internal to libphast.so.
#pragma once
#include <cstdint>
#include <vector>

#include "ch.h"

namespace phast {

enum LayoutMode : uint32_t {
    LAYOUT_WAVEFRONT = 0,   // skewed spatial wavefront (default)
    LAYOUT_LEVELS = 1,      // the paper's: level descending, input (DFS) order within a level
    LAYOUT_LEVELS_BFS = 2,  // level descending, BFS (spatial sweep) order within a level
    LAYOUT_DIAGONAL = 3,    // top levels as LEVELS_BFS, then the bottom levels in banded diagonals
};

struct Arc {
    uint32_t x, y;          // {tail, len} in G-down; {head, len} in G-up (same bytes as CUDA uint2)
};

struct Layout {
    uint32_t mode = LAYOUT_WAVEFRONT;
    uint32_t delta = 0;
    uint32_t levels = 0;
    std::vector<uint32_t> perm;      // internal_of_original
    std::vector<uint32_t> iperm;     // original_of_internal
    std::vector<uint32_t> level;     // CH level L of every internal id (0 = lowest)
    // Segments of the per-segment sweep, in processing order: [segments+1] internal-id
    // offsets; no G-down arc has both ends in one segment.  LAYOUT_LEVELS(_BFS): one
    // segment per level, j = 0 the top level.  LAYOUT_DIAGONAL: the top levels (>= cut)
    // one each, then one per diagonal.  Empty for LAYOUT_WAVEFRONT.
    std::vector<uint32_t> lvl_off;
    uint32_t cut = 0;                // LAYOUT_DIAGONAL: levels >= cut form the top part
    uint32_t lag = 1;                // LAYOUT_DIAGONAL: key(tail) <= key(head) - lag on bottom arcs
    std::vector<uint32_t> dn_first, up_first;   // [n+1]
    std::vector<Arc> dn_arc, up_arc;
    // The ORIGINAL graph's in-arcs in internal ids (parent pointers, PAPER.md:20
    // §VII-A): in_first[n+1] by head, in_arc = {tail, len} in increasing input arc
    // index per head; self-loops and length-0xFFFFFFFF arcs (never tight) dropped.
    std::vector<uint32_t> in_first;
    std::vector<Arc> in_arc;
};

// Fills L.in_first / L.in_arc from the input CSR (after layout_build).  Returns 0 or
// PHAST_ERANGE (more than 2^32-2 kept arcs).
int build_in_csr(Layout& L, uint32_t n, const uint64_t* first, const uint32_t* head, const uint32_t* len);

// Builds the renumbering from the CH result.  first/head: the input graph (used
// for the BFS that gives the spatial rank in LAYOUT_WAVEFRONT).  Returns 0,
// PHAST_ERANGE (more than 2^32-2 arcs) or PHAST_EINTERNAL (an ordering invariant
// failed: Lemma 4.1, or a G-down tail not before its head).
int layout_build(const ChResult& R, const uint64_t* first, const uint32_t* head, uint32_t mode, uint32_t delta,
                 Layout& out);

// Static schedule of the persistent sweep: the internal order is cut into chunks of
// consecutive ids (at most cap vertices; cut wherever a vertex has a G-down tail in
// the open chunk).  Chunk slot j runs on CTA j % grid in iteration j / grid.  A chunk
// whose latest tail chunk would fall in its own iteration is moved to the next
// iteration (empty pad slots in between), so every dependency points to an earlier
// iteration.  slot_v[j]..slot_v[j+1] is slot j's vertex range (empty for pads);
// dep[j] = 1 + iteration it waits for (0 = none).
struct ChunkPlan {
    std::vector<uint32_t> slot_v;   // [slots+1]
    std::vector<uint32_t> dep;      // [slots]
    uint32_t chunks = 0, slots = 0, pads = 0;
};
// cap_arcs (0 = none): also cut before a chunk's G-down arcs exceed cap_arcs;
// lag: every dependency is at least `lag` iterations earlier.
// limit (0 = n): plan only ids [0, limit) (a prefix of the order is closed under tails).
int plan_chunks(const Layout& L, uint32_t cap, uint32_t grid, ChunkPlan& out, uint32_t cap_arcs = 0,
                uint32_t lag = 1, uint32_t limit = 0);

// Warp-granular dataflow schedule (default sweep): chunks of consecutive ids (at most
// cap vertices, cut at intra-chunk dependencies), chunk c handled by worker (warp)
// c % workers in program order.  meta[4c..4c+3] = {vbeg, vend, dbeg, dend}:
// deps[dbeg..dend) are the distinct chunks holding a tail of chunk c that another
// worker handles (same-worker chunks are earlier in that worker's program order).
// Bit 31 of dend is set when chunk c depends on its worker's immediately preceding
// chunk (c - workers): a lookahead pipeline must not start chunk c before that one is
// written.  cap_arcs (0 = none) also cuts chunks before their arcs exceed it.
struct WarpPlan {
    std::vector<uint32_t> meta;
    std::vector<uint32_t> deps;
    uint32_t chunks = 0;
};
int plan_warp_chunks(const Layout& L, uint32_t cap, uint32_t workers, WarpPlan& out, uint32_t cap_arcs = 0);

// Wave schedule of the warp-wave sweep (sweep_wave_kernel).  T warps run in lock-free
// "waves": wave j is slot j*T + w of every warp w, and a wave is complete when all T
// warps have signalled it.  Chunks (consecutive ids, at most cap vertices and cap_arcs
// arcs, cut at intra-chunk arcs) are placed in increasing id order, each in the first
// wave with a free slot that is (i) after the waves of all chunks holding its tails
// and (ii) at least `window` waves below the highest wave used so far -- so the
// schedule stays close to the id order (the wavefront's L2 reuse) while a chunk never
// waits on its own wave.  Unfilled slots are empty pads.
// desc[s] = {vbeg, vcount | (dep + 1) << 8 (0: no dependency), e0 = first[vbeg], e1 = first[vbeg+vcount]}.
struct WavePlan {
    std::vector<uint32_t> desc;     // [4 * waves * T]
    uint32_t chunks = 0, waves = 0, pads = 0;
    uint64_t lag_hist[4] = {0, 0, 0, 0};   // chunks by (wave - dependency wave): 1, 2, 3, >= 4 (or none)
};
int plan_waves(const Layout& L, uint32_t cap, uint32_t cap_arcs, uint32_t T, uint32_t window, WavePlan& out);

}  // namespace phast
