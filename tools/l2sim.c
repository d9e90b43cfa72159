// LRU set-assoc cache sim of the sweep's label-row accesses in a given processing order.
#include <stdint.h>
#include <stdlib.h>
#include <stdio.h>
#include <string.h>
typedef struct { uint32_t tag; uint32_t age; } way_t;
// order[i] = old id processed i-th; newid[old] = i
uint64_t sim(uint32_t n, const uint32_t* dn_first, const uint32_t* dn_tail, const uint32_t* order,
             uint64_t cache_rows, int ways, uint64_t* reads_out, uint64_t* writes_miss) {
    uint64_t sets = cache_rows / ways;
    way_t* c = calloc(sets * ways, sizeof(way_t));
    for (uint64_t i = 0; i < sets * ways; i++) c[i].tag = 0xFFFFFFFF;
    uint32_t clock = 0; uint64_t miss = 0, reads = 0, wmiss = 0;
    uint32_t* newid = malloc((uint64_t)n * 4);
    for (uint32_t i = 0; i < n; i++) newid[order[i]] = i;
    for (uint32_t i = 0; i < n; i++) {
        uint32_t v = order[i];
        for (uint32_t e = dn_first[v]; e <= dn_first[v + 1]; e++) {
            uint32_t row; int is_write = (e == dn_first[v + 1]);
            row = is_write ? i : newid[dn_tail[e]];
            uint64_t s = ((uint64_t)row * 0x9E3779B1u) % sets;
            way_t* w = c + s * ways;
            int hit = -1, lru = 0;
            for (int j = 0; j < ways; j++) { if (w[j].tag == row) { hit = j; break; } if (w[j].age < w[lru].age) lru = j; }
            clock++;
            if (hit >= 0) { w[hit].age = clock; } else { if (!is_write) miss++; else wmiss++; w[lru].tag = row; w[lru].age = clock; }
            if (!is_write) reads++;
        }
    }
    free(c); free(newid);
    *reads_out = reads; *writes_miss = wmiss;
    return miss;
}
