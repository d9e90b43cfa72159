// ch.h -- host contraction-hierarchy preprocessor (substrate, not the optimisation
// target).  Internal to libphast.so; not part of the C ABI.
#pragma once
#include <cstdint>
#include <vector>

namespace phast {

struct ChOptions {
    uint32_t hop_limit_lo = 5;      // "5 hops up to an average degree ... of 5"  (§VIII-A)
    uint32_t hop_limit_hi = 10;     // "and by 10 hops up to degree 10"           (§VIII-A)
    uint32_t settled_cap = 1000;    // witness-search settled-vertex cap (not in the paper; safe)
    uint32_t sim_settled_cap = 0;   // cap while only estimating a priority; 0 = env PHAST_SIM_CAP or 100
    uint32_t threads = 0;           // 0 = hardware_concurrency
};

// Result of contraction: per vertex, its neighbours at the moment it was contracted
// (all of higher rank).  up_*: arcs v->x of A-up; dn_*: arcs x->v of A-down.
struct ChResult {
    uint32_t n = 0;
    std::vector<uint32_t> level;             // L(v), §IV-A level rule
    std::vector<uint32_t> rank;              // contraction round (ties: independent vertices)
    std::vector<uint64_t> up_first;          // CSR over ORIGINAL ids: arcs (v, head, len) in A-up
    std::vector<uint32_t> up_head, up_len;
    std::vector<uint64_t> dn_first;          // CSR over ORIGINAL ids: arcs (tail, v, len) in A-down, by head v
    std::vector<uint32_t> dn_tail, dn_len;
    uint32_t rounds = 0;
    double seconds = 0;
    uint64_t shortcuts = 0;
};

// first[n+1], head[m], len[m]: CSR of out-arcs.  Self-loops and arcs of length
// 0xFFFFFFFF are dropped (they can never improve a label, reading R1/R3); parallel
// arcs are merged by min.  Returns 0 or a negative phast_status.
int ch_build(uint32_t n, const uint64_t* first, const uint32_t* head, const uint32_t* len,
             const ChOptions& opt, ChResult& out);

}  // namespace phast
