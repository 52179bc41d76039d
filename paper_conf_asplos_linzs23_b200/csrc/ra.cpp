// NEXT-1: redundant-allocation pairing (§5.1 l.253-260, Fig. 3; Def 3.3
// l.154, X = 10% l.156), on the hot path's T_first / T_last.
//
// The paper's one-pass algorithm sorts every used object's first and last
// accessing API by timestamp (last after first at equal timestamps), walks the
// list from the tail to the head, and when an object's first API is reached
// (the object turns Done) recommends that it reuse the closest object to the
// left that is still Initial (its last API not yet visited) and not already
// Reused; that donor becomes Reused.  Readings R19-R21: the 10%
// size test is applied per candidate pair (|s_i - s_j|*100 <= X*max), ties go
// by object index, "closest" = the candidate whose last API is nearest to the
// left.
//
// The walk is inherently sequential (each decision changes the candidate set),
// so it runs on the host over n objects: O(n log n) with a max-segment-tree
// keyed by size rank that holds, for every candidate donor, the position of
// its last API -- a size-compatible candidate range is contiguous in size
// order, and the closest one is the range maximum.
#include <algorithm>
#include <cstdint>
#include <vector>

#include "../../include/drgpum.h"

namespace {

struct MaxTree {   // max of (position, object) over size ranks, -1 = empty
  int n = 1;
  std::vector<int64_t> t;
  explicit MaxTree(int m) { while (n < m) n <<= 1; t.assign(2 * n, -1); }
  void set(int i, int64_t v) {
    for (i += n, t[i] = v, i >>= 1; i; i >>= 1) t[i] = std::max(t[2 * i], t[2 * i + 1]);
  }
  int64_t query(int lo, int hi) const {   // max over [lo, hi)
    int64_t r = -1;
    for (lo += n, hi += n; lo < hi; lo >>= 1, hi >>= 1) {
      if (lo & 1) r = std::max(r, t[lo++]);
      if (hi & 1) r = std::max(r, t[--hi]);
    }
    return r;
  }
};

using u128 = unsigned __int128;

}  // namespace

extern "C" DRGPUM_API drgpum_status drgpum_redundant_pairs(
    const uint64_t* sizes, const uint32_t* first, const uint32_t* last, const uint8_t* used,
    uint64_t n, uint32_t pct, uint32_t* out_reuser, uint32_t* out_donor, uint64_t cap,
    uint64_t* n_pairs) {
  if (!n_pairs || (n && (!sizes || !first || !last || !used)) || pct > 100 || n >= 0x7FFFFFFFull)
    return DRGPUM_EINVAL;
  *n_pairs = 0;
  // sorted entry list: (ts, kind, obj), kind 0 = first API, 1 = last API
  struct E { uint32_t ts, kind, obj; };
  std::vector<E> ent;
  for (uint64_t o = 0; o < n; ++o)
    if (used[o]) { ent.push_back({first[o], 0u, uint32_t(o)}); ent.push_back({last[o], 1u, uint32_t(o)}); }
  std::sort(ent.begin(), ent.end(), [](const E& a, const E& b) {
    if (a.ts != b.ts) return a.ts < b.ts;
    if (a.kind != b.kind) return a.kind < b.kind;
    return a.obj < b.obj;
  });
  std::vector<int64_t> last_pos(n, -1);
  for (size_t p = 0; p < ent.size(); ++p)
    if (ent[p].kind == 1) last_pos[ent[p].obj] = int64_t(p);
  // size ranks of the used objects
  std::vector<uint32_t> by_size;
  for (uint64_t o = 0; o < n; ++o) if (used[o]) by_size.push_back(uint32_t(o));
  std::stable_sort(by_size.begin(), by_size.end(), [&](uint32_t a, uint32_t b) { return sizes[a] < sizes[b]; });
  std::vector<int> rank(n, -1);
  std::vector<uint64_t> sorted_sizes(by_size.size());
  for (size_t r = 0; r < by_size.size(); ++r) { rank[by_size[r]] = int(r); sorted_sizes[r] = sizes[by_size[r]]; }
  // every used object starts Initial: a candidate donor at its last API
  MaxTree tree(int(by_size.size()) + 1);
  const int64_t kStride = int64_t(n) + 1;   // encode (position, object) as pos*stride + obj
  for (uint64_t o = 0; o < n; ++o)
    if (used[o]) tree.set(rank[o], last_pos[o] * kStride + int64_t(o));
  const u128 X = pct, H = 100;
  for (int64_t p = int64_t(ent.size()) - 1; p >= 0; --p) {
    const E& e = ent[size_t(p)];
    if (e.kind == 1) {               // last API visited: Initial -> In Use
      tree.set(rank[e.obj], -1);
      continue;
    }
    // first API visited: Done -> the closest compatible Initial object on the left
    const u128 si = sizes[e.obj];
    // s_j < s_i: (s_i - s_j)*100 <= X*s_i  <=>  s_j*100 >= s_i*(100 - X)
    // s_j >= s_i: (s_j - s_i)*100 <= X*s_j  <=>  s_j*(100 - X) <= s_i*100
    const auto lo_it = std::partition_point(sorted_sizes.begin(), sorted_sizes.end(),
        [&](uint64_t sj) { return u128(sj) * H < si * (H - X); });
    const auto hi_it = std::partition_point(sorted_sizes.begin(), sorted_sizes.end(),
        [&](uint64_t sj) { return sj < si || u128(sj) * (H - X) <= si * H; });
    const int lo = int(lo_it - sorted_sizes.begin()), hi = int(hi_it - sorted_sizes.begin());
    if (lo >= hi) continue;
    const int64_t best = tree.query(lo, hi);
    if (best < 0) continue;
    const uint32_t donor = uint32_t(best % kStride);
    tree.set(rank[donor], -1);       // Reused: no longer available to others
    if (*n_pairs < cap) { out_reuser[*n_pairs] = e.obj; out_donor[*n_pairs] = donor; }
    ++*n_pairs;
  }
  return DRGPUM_OK;
}
