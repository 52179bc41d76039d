// NEXT-4: multi-stream dependency graph + Kahn timestamps (§5.3,
// Def 5.1 l.277-286, algorithm l.295, Fig. 4 l.291-297).
//
// Vertices are the GPU APIs in invocation order (the timestamp every access
// record carries, reading R24).  Data edges come from the attribution's
// per-(object, API) read/write sets -- the hit rows the kernels build -- so
// the graph costs O(accesses) per object instead of the paper's per-API
// shadow-memory lookups.  One left-to-right pass per object keeps the last
// writer (the ALLOC counts as one), whether any accessor followed it, and the
// readers since it; that is exactly Def 5.1's "no v_k (reads/)writes O_x
// following v_i and before v_j" conditions (R25):
//   RAW  last writer            -> every reader
//   WAR  each reader since the last write (the writer itself if it reads)
//                               -> the next writer / the FREE
//   WAW  last writer -> the next writer / the FREE, if nothing accessed O_x
//        in between.
// Kahn's algorithm (l.295 steps 1-5) then levels the DAG: every vertex of
// in-degree zero in a round gets the round's T.  Both run on the host: the
// level walk is inherently sequential along dependency chains (a single
// stream is a chain of n_api rounds), it touches O(V + E) words, and the
// expensive part -- the 1e8-record attribution that yields the read/write
// sets -- already ran on the GPU.
#include "multistream.h"

#include <algorithm>
#include <unordered_map>

namespace drgpum_ms {

void object_edges(uint32_t t_alloc, uint32_t t_free, const uint32_t* api, const uint8_t* rw,
                  size_t n, std::vector<Edge>& out) {
  uint32_t last_w = t_alloc;
  bool since = false;                  // an accessor after last_w?
  std::vector<uint32_t> readers;       // readers at or after last_w
  auto write_like = [&](uint32_t t) {
    for (uint32_t x : readers) out.push_back({x, t, DRGPUM_DEP_WAR});
    if (!since) out.push_back({last_w, t, DRGPUM_DEP_WAW});
  };
  for (size_t k = 0; k < n; ++k) {
    const uint32_t t = api[k];
    const bool r = rw[k] & 1, w = rw[k] & 2;
    if (r) out.push_back({last_w, t, DRGPUM_DEP_RAW});
    if (w) {
      write_like(t);
      last_w = t;
      since = false;
      readers.clear();
      if (r) readers.push_back(t);
    } else {
      since = true;
      readers.push_back(t);
    }
  }
  if (t_free != DRGPUM_NEVER) write_like(t_free);
}

void stream_edges(const uint32_t* stream, uint32_t n_api, std::vector<Edge>& out) {
  std::unordered_map<uint32_t, uint32_t> last;
  last.reserve(64);
  for (uint32_t v = 0; v < n_api; ++v) {
    auto it = last.find(stream[v]);
    if (it != last.end()) {
      out.push_back({it->second, v, DRGPUM_DEP_INTRA});
      it->second = v;
    } else {
      last.emplace(stream[v], v);
    }
  }
}

void canonicalize(std::vector<Edge>& e) {
  std::sort(e.begin(), e.end(), [](const Edge& a, const Edge& b) {
    return a.src != b.src ? a.src < b.src : a.dst < b.dst;
  });
  size_t m = 0;
  for (size_t i = 0; i < e.size(); ++i) {
    if (m && e[m - 1].src == e[i].src && e[m - 1].dst == e[i].dst)
      e[m - 1].label |= e[i].label;
    else
      e[m++] = e[i];
  }
  e.resize(m);
}

bool kahn(uint32_t n_api, const std::vector<Edge>& e, uint32_t* T) {
  std::vector<uint64_t> off(uint64_t(n_api) + 1, 0);   // CSR by src (e sorted by src)
  std::vector<uint32_t> indeg(n_api, 0);
  for (const Edge& x : e) { ++off[x.src + 1]; ++indeg[x.dst]; }
  for (uint32_t v = 0; v < n_api; ++v) off[v + 1] += off[v];
  std::vector<uint32_t> cur, nxt;
  for (uint32_t v = 0; v < n_api; ++v)                 // (1) T = 0, (2) in-degree zero
    if (!indeg[v]) cur.push_back(v);
  uint32_t t = 0, done = 0;
  while (!cur.empty()) {                               // (5) until the graph is empty
    for (uint32_t v : cur) T[v] = t;                   // (2) annotate
    done += uint32_t(cur.size());
    nxt.clear();
    for (uint32_t v : cur)                             // (2) delete, (3) update in-degrees
      for (uint64_t k = off[v]; k < off[v + 1]; ++k)
        if (--indeg[e[k].dst] == 0) nxt.push_back(e[k].dst);
    cur.swap(nxt);
    ++t;                                               // (4)
  }
  return done == n_api;
}

}  // namespace drgpum_ms

extern "C" DRGPUM_API drgpum_status drgpum_kahn_levels(uint32_t n_api, const uint32_t* src,
                                                        const uint32_t* dst, uint64_t n_edges,
                                                        uint32_t* h_T) {
  if ((n_api && !h_T) || (n_edges && (!src || !dst))) return DRGPUM_EINVAL;
  std::vector<drgpum_ms::Edge> e(n_edges);
  for (uint64_t k = 0; k < n_edges; ++k) {
    if (src[k] >= n_api || dst[k] >= n_api) return DRGPUM_EINVAL;
    e[k] = {src[k], dst[k], 0};
  }
  drgpum_ms::canonicalize(e);
  return drgpum_ms::kahn(n_api, e, h_T) ? DRGPUM_OK : DRGPUM_EINVAL;
}
