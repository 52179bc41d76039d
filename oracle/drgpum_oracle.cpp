// DrGPUM per-access object attribution -- the CPU ORACLE (O1).
//
// TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and
// bench.py's cpu_baseline / --impl reference legs may load this library.  The
// product path (paper_conf_asplos_linzs23_b200) never imports, links or calls
// anything under oracle/, and this file shares no code, header, table or
// helper with paper_conf_asplos_linzs23_b200/csrc.  Its struct layouts are
// retyped here from the interchange format; they are data
// formats, not code.
//
// What it computes, and where the paper defines it ("P:NNN" = line of
// /root/reference/PAPER.md):
//   * the memory map M: insert the address range of each object at its
//     allocation API, remove it at its deallocation API, look it up at every
//     memory copy / set / kernel launch (§5.1);
//   * timestamps T aligned with invocation order (§5.1);
//   * per-object bitmap, one bit per element, set to 1 on access (P:266-268,
//     §5.2 "Overallocation");
//   * T_first / T_last and the list of GPU APIs that access each object
//     (§5.1; Fig. 2);
//   * the object-level rules EA, LD, UA, ML, TI, DW (Defs 3.1-3.7
//     P:124-170) and the intra-object rule OA with Frag, Eq. (1) (P:174,
//     P:189-194).
// It is deliberately slow and literal: a std::map replay of the whole
// timeline, one bit set at a time, linear scans for every reduction.
// Readings of the paper where it is silent or ambiguous are the numbered
// items of DESIGN.md §"Readings" (R1..R18), cited below as [Rn].
//
// Parity pins: tests/test_oracle_pins.py (paper worked examples, closed forms,
// invariants) and tests/test_bruteforce.py (O0, a literal per-definition brute
// force in Python).  No function here is "parity unpinned".

#include <cstdint>
#include <cstring>
#include <map>
#include <set>
#include <vector>
#include <algorithm>

namespace {

enum : uint32_t { K_ALLOC = 0, K_FREE = 1, K_MEMCPY = 2, K_MEMSET = 3, K_KERNEL = 4 };
const uint32_t NEVER_T = 0xFFFFFFFFu;
enum : int { S_OK = 0, S_EINVAL = 1, S_EOVERLAP = 2 };

struct Obj { uint64_t base, size; uint32_t elem_size, t_alloc, t_free, user_id; };
struct Rec { uint64_t addr; uint32_t size, meta; };
struct Stats {
  uint64_t n_elems, accessed, span_lo, span_hi, largest_unaccessed_run;
  uint32_t t_first, t_last, n_access_apis, pad;
};
struct Thresholds { uint32_t ti_min_idle, oa_accessed_pct, oa_frag_pct; };
struct Report {
  uint32_t flags, ea_distance, ld_distance, ti_ranges, ti_max_idle, dw_pairs;
  uint64_t ti_total_idle;
};
struct Counters { uint64_t records, attributed, unattributed, clipped, invalid; };

enum : uint32_t { F_EA = 1, F_LD = 2, F_UA = 4, F_ML = 8, F_TI = 16, F_DW = 32,
                  F_OA = 64, F_OA_ACT = 128 };

struct Flags { bool read, write; };

struct State {
  std::vector<Obj> objs;
  std::vector<uint8_t> kinds;
  std::vector<std::vector<bool>> bitmap;       // one bit per element
  std::vector<uint32_t> first, last;           // T_first, T_last
  std::vector<std::map<uint32_t, Flags>> accesses;  // APIs that access O, by T
  Counters ctr;
  std::vector<std::vector<uint32_t>> alloc_at, free_at;   // per timestamp
  // NEXT-3 structured access (Def 3.10; §5.2 l.270 "multiple bitmaps for a
  // data object, where each bitmap represents memory accesses of a GPU API"):
  // per (object, API) the set of elements that API touched
  std::map<std::pair<uint32_t, uint32_t>, std::set<uint64_t>> api_elems;
  bool track_sa = false;
  // NEXT-2 non-uniform access frequency (Def 3.9, l.271): per (object, API)
  // the "hashmap" of element -> access frequency of that API
  std::map<std::pair<uint32_t, uint32_t>, std::map<uint64_t, uint64_t>> freq;
  bool track_freq = false;
};

}  // namespace

extern "C" {

// Validation (SURVEY §8(b) rules; [R5], [R13]).  Returns S_OK / S_EINVAL /
// S_EOVERLAP and the index of the first offending object (or UINT64_MAX).
int oracle_validate(const Obj* objs, uint64_t n_obj, const uint8_t* kinds,
                    uint32_t n_api, uint64_t* bad) {
  *bad = UINT64_MAX;
  if (n_api >= 0x80000000u) return S_EINVAL;
  if (n_obj >= 0xFFFFFFFFull) return S_EINVAL;
  for (uint32_t t = 0; t < n_api; ++t)
    if (kinds[t] > K_KERNEL) return S_EINVAL;
  for (uint64_t i = 0; i < n_obj; ++i) {
    const Obj& o = objs[i];
    const uint32_t E = o.elem_size;
    bool ok = o.size != 0 && (E == 1 || E == 2 || E == 4 || E == 8 || E == 16) &&
              o.size % E == 0 && o.base <= UINT64_MAX - o.size &&
              o.t_alloc < n_api && kinds[o.t_alloc] == K_ALLOC;
    if (ok && o.t_free != NEVER_T)
      ok = o.t_free < n_api && o.t_free > o.t_alloc && kinds[o.t_free] == K_FREE;
    if (!ok) { *bad = i; return S_EINVAL; }
  }
  // Overlap: replay allocations/frees through M; an insert that meets a live
  // entry with an intersecting address range means two objects overlap in
  // address and in (open) lifetime.  [R5]
  std::vector<std::vector<uint64_t>> at_alloc(n_api), at_free(n_api);
  for (uint64_t i = 0; i < n_obj; ++i) {
    at_alloc[objs[i].t_alloc].push_back(i);
    if (objs[i].t_free != NEVER_T) at_free[objs[i].t_free].push_back(i);
  }
  std::map<uint64_t, uint64_t> M;  // base -> object
  for (uint32_t t = 0; t < n_api; ++t) {
    for (uint64_t i : at_free[t]) M.erase(objs[i].base);
    for (uint64_t i : at_alloc[t]) {
      const uint64_t b = objs[i].base, e = b + objs[i].size;
      auto it = M.lower_bound(b);
      if (it != M.end() && it->first < e) { *bad = i; return S_EOVERLAP; }
      if (it != M.begin()) {
        auto p = std::prev(it);
        if (objs[p->second].base + objs[p->second].size > b) { *bad = i; return S_EOVERLAP; }
      }
      M[b] = i;
    }
  }
  return S_OK;
}

void* oracle_new(const Obj* objs, uint64_t n_obj, const uint8_t* kinds,
                 uint32_t n_api, int* status) {
  uint64_t bad;
  *status = oracle_validate(objs, n_obj, kinds, n_api, &bad);
  if (*status != S_OK) return nullptr;
  State* s = new State();
  s->objs.assign(objs, objs + n_obj);
  s->kinds.assign(kinds, kinds + n_api);
  s->bitmap.resize(n_obj);
  for (uint64_t i = 0; i < n_obj; ++i)
    s->bitmap[i].assign(objs[i].size / objs[i].elem_size, false);  // "untouched" (0)
  s->first.assign(n_obj, NEVER_T);
  s->last.assign(n_obj, 0);
  s->accesses.resize(n_obj);
  std::memset(&s->ctr, 0, sizeof(s->ctr));
  s->alloc_at.resize(n_api);
  s->free_at.resize(n_api);
  for (uint64_t i = 0; i < n_obj; ++i) {
    s->alloc_at[objs[i].t_alloc].push_back((uint32_t)i);
    if (objs[i].t_free != NEVER_T) s->free_at[objs[i].t_free].push_back((uint32_t)i);
  }
  return s;
}

void oracle_free(void* p) { delete static_cast<State*>(p); }

// NEXT-3: record, for every element, which GPU APIs touch it (call before
// oracle_attribute).
void oracle_track_structured(void* p) {
  State& s = *static_cast<State*>(p);
  s.track_sa = true;
  s.api_elems.clear();
}

// NEXT-2: keep, per (object, GPU API), the access frequency of every element
// that API touches (call before oracle_attribute).
void oracle_track_frequency(void* p) {
  static_cast<State*>(p)->track_freq = true;
}

// NEXT-2 non-uniform access frequency (Def 3.9 l.196; §5.2 l.271; fn 3 l.222:
// coefficient of variation).  For every (object O, accessing API A): n =
// number of elements A touched (cells of A's hashmap for O), S1 = sum of
// their frequencies, S2 = sum of squares.  Rows are written in (object, ts)
// order: obj[k], ts[k], n[k], s1[k], s2[k]; returns the number of rows.
uint64_t oracle_frequency(void* p, uint32_t* obj, uint32_t* ts, uint64_t* n, uint64_t* s1,
                          uint64_t* s2, uint64_t cap) {
  State& s = *static_cast<State*>(p);
  uint64_t k = 0;
  for (const auto& kv : s.freq) {
    if (k < cap) {
      uint64_t a = 0, b = 0;
      for (const auto& ec : kv.second) { a += ec.second; b += ec.second * ec.second; }
      obj[k] = kv.first.first;
      ts[k] = kv.first.second;
      n[k] = kv.second.size();
      s1[k] = a;
      s2[k] = b;
    }
    ++k;
  }
  return k;
}

// NEXT-3 structured access (Def 3.10, l.200; §5.2 l.270): object O matches if
// each GPU API that accesses it touches a slice of O and the slices do not
// overlap -- the per-API bitmaps of O are pairwise disjoint, and at least two
// APIs access O.  [R23] The APIs considered are those with in_group[t] != 0
// (NULL = every API): the paper reports the pattern "at GPU kernel
// gramschmidt_kernel3" (l.400), i.e. over the invocations of one kernel.
// out[o] = 1 if O matches; overlap[o] = 1 if two of those APIs share an element.
void oracle_structured_group(void* p, const uint8_t* in_group, uint8_t* out, uint8_t* overlap) {
  State& s = *static_cast<State*>(p);
  const size_t n = s.objs.size();
  std::vector<uint64_t> n_api(n, 0), sum(n, 0);
  std::vector<std::set<uint64_t>> uni(n);
  for (const auto& kv : s.api_elems) {
    const uint32_t o = kv.first.first, t = kv.first.second;
    if (in_group && !in_group[t]) continue;
    n_api[o]++;
    sum[o] += kv.second.size();
    uni[o].insert(kv.second.begin(), kv.second.end());
  }
  for (size_t o = 0; o < n; ++o) {
    const bool ov = uni[o].size() < sum[o];      // some element is in two APIs' bitmaps
    overlap[o] = ov ? 1 : 0;
    out[o] = (n_api[o] >= 2 && !ov) ? 1 : 0;
  }
}

void oracle_structured(void* p, uint8_t* out, uint8_t* overlap) {
  oracle_structured_group(p, nullptr, out, overlap);
}

// Slice-level access frequency (Def 3.9 l.196 read at the granularity of
// l.400: "the variance of access frequencies of individual slices in R_gpu is
// 58%") [R22b]: for object O and the APIs with in_group[t] != 0, the access
// frequency of API A's slice is F_A = the sum of the element frequencies of
// A's hashmap for O (l.271).  out[4o..4o+3] = { n = number of such APIs that
// access O, sum F_A, and sum F_A^2 as (low 64 bits, high 64 bits) }.  Needs
// oracle_track_frequency.
void oracle_slice_frequency(void* p, const uint8_t* in_group, uint64_t* out) {
  State& s = *static_cast<State*>(p);
  const size_t n = s.objs.size();
  std::vector<unsigned __int128> s2(n, 0);
  for (size_t o = 0; o < n; ++o) out[4 * o] = out[4 * o + 1] = 0;
  for (const auto& kv : s.freq) {
    const uint32_t o = kv.first.first, t = kv.first.second;
    if (in_group && !in_group[t]) continue;
    uint64_t F = 0;
    for (const auto& ec : kv.second) F += ec.second;
    out[4 * o] += 1;
    out[4 * o + 1] += F;
    s2[o] += (unsigned __int128)F * F;
  }
  for (size_t o = 0; o < n; ++o) {
    out[4 * o + 2] = (uint64_t)s2[o];
    out[4 * o + 3] = (uint64_t)(s2[o] >> 64);
  }
}

// Attribute n records.  May be called repeatedly (chunks); each call replays
// the timeline over its own records.  Records are grouped by timestamp first
// (stable counting sort) so that every record is looked up in M as M stands
// at its API's invocation.
void oracle_attribute(void* p, const Rec* recs, uint64_t n) {
  State& s = *static_cast<State*>(p);
  const uint32_t n_api = (uint32_t)s.kinds.size();
  s.ctr.records += n;
  // A1: invalid records are counted and ignored ([R14]).
  std::vector<uint64_t> count(n_api + 1, 0);
  std::vector<uint8_t> valid(n, 0);
  for (uint64_t i = 0; i < n; ++i) {
    const uint32_t ts = recs[i].meta & 0x7FFFFFFFu;
    const bool ok = recs[i].size != 0 && ts < n_api && s.kinds[ts] != K_ALLOC &&
                    s.kinds[ts] != K_FREE && recs[i].addr <= UINT64_MAX - recs[i].size;
    if (!ok) { s.ctr.invalid++; continue; }
    valid[i] = 1;
    count[ts + 1]++;
  }
  for (uint32_t t = 0; t < n_api; ++t) count[t + 1] += count[t];
  std::vector<uint64_t> order(count[n_api]);
  {
    std::vector<uint64_t> pos(count.begin(), count.end() - 1);
    for (uint64_t i = 0; i < n; ++i)
      if (valid[i]) order[pos[recs[i].meta & 0x7FFFFFFFu]++] = i;
  }
  std::map<uint64_t, uint32_t> M;  // memory map: start address -> object
  for (uint32_t t = 0; t < n_api; ++t) {
    if (s.kinds[t] == K_ALLOC) {
      for (uint32_t o : s.alloc_at[t]) M[s.objs[o].base] = o;
      continue;
    }
    if (s.kinds[t] == K_FREE) {
      for (uint32_t o : s.free_at[t]) M.erase(s.objs[o].base);
      continue;
    }
    for (uint64_t k = count[t]; k < count[t + 1]; ++k) {
      const Rec& r = recs[order[k]];
      const bool is_write = (r.meta >> 31) != 0;
      auto it = M.upper_bound(r.addr);
      if (it == M.begin()) { s.ctr.unattributed++; continue; }        // [R4]
      --it;
      const uint32_t o = it->second;
      const Obj& ob = s.objs[o];
      const uint64_t obj_end = ob.base + ob.size;
      if (r.addr >= obj_end) { s.ctr.unattributed++; continue; }      // [R4]
      s.ctr.attributed++;
      uint64_t end = r.addr + r.size;
      if (end > obj_end) { end = obj_end; s.ctr.clipped++; }          // [R3]
      // which element(s) the access touches; partial touch counts [R2]
      const uint64_t e0 = (r.addr - ob.base) / ob.elem_size;
      const uint64_t e1 = (end - 1 - ob.base) / ob.elem_size;
      for (uint64_t e = e0; e <= e1; ++e) s.bitmap[o][e] = true;
      if (s.track_freq) {                                             // l.271
        auto& hm = s.freq[{o, t}];
        for (uint64_t e = e0; e <= e1; ++e) hm[e] += 1;
      }
      if (s.track_sa) {                                               // l.270
        auto& bm = s.api_elems[{o, t}];
        for (uint64_t e = e0; e <= e1; ++e) bm.insert(e);
      }
      if (t < s.first[o]) s.first[o] = t;
      if (t > s.last[o]) s.last[o] = t;
      Flags& f = s.accesses[o][t];   // value-initialised {false, false} on first touch
      if (is_write) f.write = true; else f.read = true;
    }
  }
}

// Per-object statistics ("examines each data object's bitmap to compute
// the percentage of accessed elements"; Eq. (1) P:191 needs the largest
// unaccessed chunk).  Linear scans, one element at a time.
void oracle_stats(void* p, Stats* out, Counters* ctr) {
  State& s = *static_cast<State*>(p);
  for (size_t o = 0; o < s.objs.size(); ++o) {
    const auto& bm = s.bitmap[o];
    Stats st;
    std::memset(&st, 0, sizeof(st));
    st.n_elems = bm.size();
    st.span_lo = UINT64_MAX;
    st.span_hi = UINT64_MAX;
    uint64_t run = 0;
    for (uint64_t e = 0; e < bm.size(); ++e) {
      if (bm[e]) {
        st.accessed++;
        if (st.span_lo == UINT64_MAX) st.span_lo = e;
        st.span_hi = e;
        run = 0;
      } else {
        run++;
        if (run > st.largest_unaccessed_run) st.largest_unaccessed_run = run;
      }
    }
    st.t_first = s.first[o];
    st.t_last = s.last[o];
    st.n_access_apis = (uint32_t)s.accesses[o].size();
    out[o] = st;
  }
  *ctr = s.ctr;
}

// Pattern rules, in exact integer arithmetic.
//   "between" = strictly between, over all GPU APIs including alloc/free/set
//   [R6]: the number of APIs between timestamps a < b is b - a - 1 in the
//   dense single-stream timeline.
void oracle_patterns(void* p, const Thresholds* th, Report* out) {
  State& s = *static_cast<State*>(p);
  for (size_t o = 0; o < s.objs.size(); ++o) {
    const Obj& ob = s.objs[o];
    // the accessing APIs a_1 < ... < a_k of O (std::map iterates in T order)
    std::vector<uint32_t> ts;
    std::vector<Flags> fl;
    for (const auto& kv : s.accesses[o]) { ts.push_back(kv.first); fl.push_back(kv.second); }
    Report r;
    std::memset(&r, 0, sizeof(r));
    const bool used = !ts.empty();
    const bool leak = ob.t_free == NEVER_T;
    if (!used) r.flags |= F_UA;                                        // Def 3.4
    if (leak) r.flags |= F_ML;                                         // Def 3.5
    if (used) {
      const uint32_t first = ts.front(), last = ts.back();
      if (first - ob.t_alloc - 1 >= 1) {                               // Def 3.1 [R7]
        r.flags |= F_EA;
        r.ea_distance = first - ob.t_alloc;
      }
      if (!leak && ob.t_free - last - 1 >= 1) {                        // Def 3.2 [R8]
        r.flags |= F_LD;
        r.ld_distance = ob.t_free - last;
      }
      for (size_t i = 0; i + 1 < ts.size(); ++i) {
        const uint32_t gap = ts[i + 1] - ts[i] - 1;                    // Def 3.6
        if (gap >= th->ti_min_idle) {
          r.ti_ranges++;
          if (gap > r.ti_max_idle) r.ti_max_idle = gap;
          r.ti_total_idle += gap;
        }
        const uint8_t ka = s.kinds[ts[i]], kb = s.kinds[ts[i + 1]];
        const bool cs_a = ka == K_MEMCPY || ka == K_MEMSET;
        const bool cs_b = kb == K_MEMCPY || kb == K_MEMSET;
        if (cs_a && cs_b && fl[i].write && fl[i + 1].write) r.dw_pairs++;    // Def 3.7 [R12]
      }
      if (r.ti_ranges) r.flags |= F_TI;
      if (r.dw_pairs) r.flags |= F_DW;
    }
    // Def 3.8 with "less than X%" strict [R10]; Eq. (1) Frag < X_frag [R11].
    const auto& bm = s.bitmap[o];
    uint64_t accessed = 0, run = 0, cur = 0;
    for (bool b : bm) {
      if (b) { accessed++; cur = 0; } else { cur++; if (cur > run) run = cur; }
    }
    const uint64_t n = bm.size();
    if (100 * accessed < (uint64_t)th->oa_accessed_pct * n) {
      r.flags |= F_OA;
      const uint64_t unacc = n - accessed;
      if (unacc == 0 || 100 * (unacc - run) < (uint64_t)th->oa_frag_pct * unacc)
        r.flags |= F_OA_ACT;
    }
    out[o] = r;
  }
}

// Export helpers for the parity tests.
// Bitmap of object o, packed LSB-first into ceil(n_elem/8) bytes.
void oracle_get_bitmap(void* p, uint64_t o, uint8_t* out) {
  State& s = *static_cast<State*>(p);
  const auto& bm = s.bitmap[o];
  std::memset(out, 0, (bm.size() + 7) / 8);
  for (uint64_t e = 0; e < bm.size(); ++e)
    if (bm[e]) out[e >> 3] |= (uint8_t)(1u << (e & 7));
}

// The APIs that access object o: timestamps and flags (bit0 read, bit1 write).
uint64_t oracle_get_accesses(void* p, uint64_t o, uint32_t* ts, uint8_t* rw, uint64_t cap) {
  State& s = *static_cast<State*>(p);
  const auto& acc = s.accesses[o];
  uint64_t i = 0;
  for (const auto& kv : acc) {
    if (i >= cap) break;
    ts[i] = kv.first;
    rw[i] = (uint8_t)((kv.second.read ? 1 : 0) | (kv.second.write ? 2 : 0));
    ++i;
  }
  return acc.size();
}

}  // extern "C"
