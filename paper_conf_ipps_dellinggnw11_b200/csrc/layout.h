// layout.h -- vertex renumbering and the G-up / G-down CSRs in internal ids.
// Internal to libphast.so.
#pragma once
#include <cstdint>
#include <vector>

#include "ch.h"

namespace phast {

enum LayoutMode : uint32_t {
    LAYOUT_LEVELS = 1,      // the paper's: level descending, input (DFS) order within a level
    LAYOUT_LEVELS_BFS = 2,  // level descending, BFS (spatial sweep) order within a level
    LAYOUT_LEVELS_BANDS = 3,  // LEVELS_BFS, with the bottom levels cut into bands of closed groups (default)
};

// A band: consecutive levels (segments [seg_lo, seg_hi) in processing order) whose
// vertices are partitioned into GROUPS closed under the band's own G-down arcs: an
// arc (u, v) with both ends in the band has both ends in one group.  A group only
// needs rows from above the band and from itself, so groups are independent work
// (band_kernel, sweep.cu).  Within each level of the band, vertices are sorted by
// group (then BFS rank), so group g of segment j is the contiguous id range
// [goff[(j - seg_lo) * (ngroups + 1) + g], goff[... + g + 1]).  Groups are formed from
// the connected components of the band's arcs in BFS-rank order, each group at least
// BAND_GROUP_MIN vertices (the last may be smaller).
struct Band {
    uint32_t seg_lo = 0, seg_hi = 0, ngroups = 0;
    std::vector<uint32_t> goff;   // [(seg_hi - seg_lo) * (ngroups + 1)]
};
constexpr uint32_t BAND_GROUP_MIN = 32;
// a band grows upward while its largest component has at most this many vertices and
// at most 1 / BAND_COMP_DIV of the band's vertices (one component is one CTA's serial
// work: C3 k = 64, a 942-vertex component in a 2 764-vertex band took 55 us against 24
// for its four per-level launches)
constexpr uint32_t BAND_COMP_CAP = 1024;
constexpr uint32_t BAND_COMP_DIV = 256;
// ... and has at most this many levels (BandArgs::wide is a 32-bit mask)
constexpr uint32_t BAND_MAX_LEVELS = 32;

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
    // LAYOUT_LEVELS_BANDS: the bands, top-most first (their segments are the last ones)
    std::vector<Band> bands;
};

// Checks the band invariants of L (group ranges tile each band level in order; every
// G-down arc inside a band stays inside one group).  Returns 0 or PHAST_EINTERNAL.
int check_bands(const Layout& L);

// Fills L.in_first / L.in_arc from the input CSR (after layout_build).  Returns 0 or
// PHAST_ERANGE (more than 2^32-2 kept arcs).
int build_in_csr(Layout& L, uint32_t n, const uint64_t* first, const uint32_t* head, const uint32_t* len);

// Builds the renumbering from the CH result.  first/head: the input graph (used for
// the BFS that gives the spatial rank in LAYOUT_LEVELS_BFS).  Returns 0, PHAST_EINVAL
// (unknown mode), PHAST_ERANGE (more than 2^32-2 arcs) or PHAST_EINTERNAL (an ordering
// invariant failed: Lemma 4.1, or a G-down tail not before its head).
int layout_build(const ChResult& R, const uint64_t* first, const uint32_t* head, uint32_t mode, Layout& out);

}  // namespace phast
