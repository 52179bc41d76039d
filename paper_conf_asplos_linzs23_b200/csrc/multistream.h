// NEXT-4 (§5.3): dependency graph (Def 5.1) and Kahn timestamps.
// Host-side algorithms shared by the drgpum_dependency_graph /
// drgpum_patterns_topo entry points in host.cpp.
#pragma once
#include <cstdint>
#include <vector>

#include "../../include/drgpum.h"

namespace drgpum_ms {

struct Edge {
  uint32_t src, dst;
  uint32_t label;   // DRGPUM_DEP_* bits
};

// One object's accesses in invocation order: api[k], rw[k] (bit0 read, bit1
// write).  Appends its RAW / WAW / WAR edges (Def 5.1 l.283-285).
void object_edges(uint32_t t_alloc, uint32_t t_free, const uint32_t* api, const uint8_t* rw,
                  size_t n, std::vector<Edge>& out);

// Intra-stream immediate successors (Def 5.1 l.281).
void stream_edges(const uint32_t* stream, uint32_t n_api, std::vector<Edge>& out);

// Sort by (src, dst) and merge duplicates (labels OR-ed).
void canonicalize(std::vector<Edge>& e);

// Kahn levels (l.295) over edges sorted by src.  false on a cycle.
bool kahn(uint32_t n_api, const std::vector<Edge>& e, uint32_t* T);

}  // namespace drgpum_ms
