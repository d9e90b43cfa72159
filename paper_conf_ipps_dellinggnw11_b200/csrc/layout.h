// layout.h -- vertex renumbering and the G-up / G-down CSRs in internal ids.
// Internal to libphast.so.
#pragma once
#include <cstdint>
#include <vector>

#include "ch.h"

namespace phast {

enum LayoutMode : uint32_t {
    LAYOUT_LEVELS = 1,      // the paper's: level descending, input (DFS) order within a level
    LAYOUT_LEVELS_BFS = 2,  // level descending, BFS (spatial sweep) order within a level (default)
};

struct Arc {
    uint32_t x, y;          // {tail, len} in G-down; {head, len} in G-up (same bytes as CUDA uint2)
};

struct Layout {
    uint32_t mode = LAYOUT_LEVELS_BFS;
    uint32_t levels = 0;
    std::vector<uint32_t> perm;      // internal_of_original
    std::vector<uint32_t> iperm;     // original_of_internal
    std::vector<uint32_t> level;     // CH level L of every internal id (0 = lowest)
    // Level offsets in processing order: [levels+1] internal ids, j = 0 the top level;
    // no G-down arc has both ends in one level (Lemma 4.1).
    std::vector<uint32_t> lvl_off;
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

// Builds the renumbering from the CH result.  first/head: the input graph (used for
// the BFS that gives the spatial rank in LAYOUT_LEVELS_BFS).  Returns 0, PHAST_EINVAL
// (unknown mode), PHAST_ERANGE (more than 2^32-2 arcs) or PHAST_EINTERNAL (an ordering
// invariant failed: Lemma 4.1, or a G-down tail not before its head).
int layout_build(const ChResult& R, const uint64_t* first, const uint32_t* head, uint32_t mode, Layout& out);

}  // namespace phast
