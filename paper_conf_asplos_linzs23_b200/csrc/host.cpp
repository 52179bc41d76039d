// Host side of libdrgpum.so: validation, the static segment index that
// replaces DrGPUM's memory map M, workspace layout, and the C ABI.
//
// M (§5.1 l.238-240) maps the address range of every ACTIVE object
// to the object and is updated at every alloc/free.  For a whole recorded
// trace the library builds it once, for all timestamps at the same time: the
// address line is cut at every object boundary into elementary segments, and
// each segment lists the objects covering it sorted by t_alloc.  Because two
// objects may not overlap in address and lifetime (reading R5), the object
// live at ts in a segment is the last candidate with t_alloc < ts, provided
// ts < its t_free.  With no address reuse every segment has at most one
// candidate and the lookup is exactly the paper's binary search over M
// (l.322, Fig. 5).  Validation of R5 falls out of the same structure: the
// sorted candidates of every segment must have disjoint open lifetimes.
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdarg>
#include <cstdio>
#include <cstring>
#include <numeric>
#include <string>
#include <vector>

#include "../../include/drgpum.h"
#include "internal.cuh"
#include "multistream.h"

using namespace drgpum;

namespace {
enum State { S_CREATED = 0, S_LOADED = 1, S_BOUND = 2 };

struct Layout {
  uint64_t orw, first, last, ctr, cons;     // dynamic (reset per trace)
  uint64_t pmask;
  uint64_t dyn_end;
  uint64_t objs, seg_start, seg_cand_off, seg, cand, l1, acc_rank, acc_ts, acc_cs, n_hit;
  uint64_t rfull;                 // per object: a whole-object range was queued in this trace
  uint64_t tiles, tile_part, groups, group_off, group_part, stats, reports, rq, stage, hints;
  // NEXT-3 structured access (feature): owner[sum n_elem], overlap[n_obj], elem_base, queue
  uint64_t sa_owner, sa_overlap, sa_elem_base, sa_q, sa_qcount, sa_end, sa_group;
  // NEXT-2 frequency (feature): cells[sum n_elem], acc[n_slots][3], state, queue, outputs
  uint64_t fq_acc, fq_state, fq_ctl, fq_end, fq_acc_q, fq_slot_base, fq_out_count, fq_out_first;
  uint64_t fq_keys0, fq_keys1, fq_hist, fq_offs, fq_part;
  uint64_t total;
};

constexpr uint64_t kAlign = 256;
inline uint64_t align_up(uint64_t x, uint64_t a = kAlign) { return (x + a - 1) / a * a; }
}  // namespace

struct drgpum_ctx {
  int device = 0;
  int num_sms = 148;
  int attr_occ = 1;   // blocks per SM of the persistent attribution kernel, on this device
  State state = S_CREATED;
  std::string err;
  uint64_t launches = 0;
  // program
  uint64_t n_obj = 0;
  uint32_t n_api = 0, n_acc = 0;
  std::vector<drgpum_object_t> objs;
  std::vector<uint8_t> kinds;
  // derived tables (uploaded at bind)
  std::vector<DevObj> dobj;
  std::vector<uint64_t> seg_start;
  std::vector<uint32_t> seg_cand_off;
  std::vector<SegEntry> seg;
  std::vector<CandEntry> cand;
  std::vector<uint64_t> l1;
  uint32_t l1_stride = 1;
  std::vector<uint32_t> acc_rank, acc_ts, n_hit;
  std::vector<uint8_t> acc_cs;
  std::vector<Tile> tiles;
  std::vector<uint32_t> tile_off;
  std::vector<Group> groups;
  std::vector<uint32_t> group_off;
  std::vector<uint64_t> small_prefix;   // finalize: prefix count of lane-foldable objects
  uint64_t n_small_tiles = 0;           // tiles of <= 128 words (the sparse reset's lane mode)
  std::vector<drgpum_object_layout_t> layout;
  uint64_t bitmap_words = 0, hit_words = 0;
  uint32_t rq_cap = 1u << 20;
  uint64_t attr_calls = 0;        // parity selects the range-queue count slot
  uint32_t features = 0;
  std::vector<uint64_t> elem_base, slot_base;
  uint64_t n_elem_total = 0, n_slots = 0;
  uint32_t sa_q_cap = 1u << 20;
  uint64_t fq_recs = 1ull << 24;   // NEXT-2: records per frequency sub-call
  uint32_t fq_pos_bits = 1, fq_digits = 1;
  std::vector<uint8_t> api_group;   // NEXT-2/3 API group [R22b, R23] (1 = in), mirrored in the workspace
  Layout L{};
  uint8_t* ws = nullptr;
  uint64_t ws_bytes = 0;
  // finalize cache
  bool final_valid = false;
  drgpum_thresholds_t final_th{2, 80, 80};
  // owned merge: this rank holds the merged shadow of objects [own_lo, own_hi) only
  bool owned = false, gathered = false;
  // reduce-and-clear (drgpum_set_finalize_consume): finalize zeroes the
  // bitmap words it reduces; consumed = they are zero and the tile monoids
  // are authoritative until the next reset
  bool fin_consume = false, consumed = false;
  uint64_t own_lo = 0, own_hi = 0;
  uint32_t own_P = 0, own_rank = 0;
  // host ingest
  cudaStream_t copy_stream = nullptr;
  cudaEvent_t ev_copied[2] = {nullptr, nullptr}, ev_used[2] = {nullptr, nullptr};
};

namespace {

drgpum_status fail(drgpum_ctx* c, drgpum_status s, const char* fmt, ...) {
  char buf[512];
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(buf, sizeof buf, fmt, ap);
  va_end(ap);
  if (c) c->err = buf;
  return s;
}

drgpum_status cuda_check(drgpum_ctx* c, cudaError_t e, const char* what) {
  if (e == cudaSuccess) return DRGPUM_OK;
  return fail(c, DRGPUM_ECUDA, "%s: %s", what, cudaGetErrorString(e));
}

#define CK(expr)                                                     \
  do {                                                               \
    drgpum_status _s = cuda_check(ctx, (expr), #expr);               \
    if (_s != DRGPUM_OK) return _s;                                  \
  } while (0)

template <typename T> T* at(drgpum_ctx* c, uint64_t off) { return reinterpret_cast<T*>(c->ws + off); }

cudaStream_t as_stream(void* s) { return reinterpret_cast<cudaStream_t>(s); }

// Every launching / copying entry point runs on the context's device,
// whichever device the calling thread has current.
drgpum_status set_device(drgpum_ctx* ctx) {
  int cur = -1;
  if (cudaGetDevice(&cur) == cudaSuccess && cur == ctx->device) return DRGPUM_OK;
  CK(cudaSetDevice(ctx->device));
  return DRGPUM_OK;
}

uint32_t ilog2(uint32_t e) { uint32_t s = 0; while ((1u << s) < e) ++s; return s; }

drgpum_status compute_layout(drgpum_ctx* c);
drgpum_status gather_accesses(drgpum_ctx* ctx, cudaStream_t st, std::vector<uint64_t>& off,
                              std::vector<uint32_t>& api, std::vector<uint8_t>& rw);

// NEXT-2 event-key capacity: two keys per record of a sub-call (records of
// one attribute call are processed in sub-calls of at most fq_recs) plus
// the carried keys of an API that continues across (sub-)calls.
uint64_t freq_cap(const drgpum_ctx* c) { return 3 * c->fq_recs; }
uint64_t freq_max_tiles(const drgpum_ctx* c) { return (freq_cap(c) + kFreqTileKeys - 1) / kFreqTileKeys; }
uint32_t bits_for(uint64_t v) { uint32_t b = 0; while (b < 64 && (v >> b)) ++b; return b; }

// Build everything derived from (objects, kinds) on the host.
drgpum_status build_tables(drgpum_ctx* c) {
  const uint64_t n = c->n_obj;
  const uint32_t n_api = c->n_api;
  // access-API ranks (footnote 2, l.178: ALLOC/FREE never access)
  c->acc_rank.assign(n_api, kNone);
  c->acc_ts.clear();
  c->acc_cs.clear();
  std::vector<uint32_t> acc_before(uint64_t(n_api) + 1, 0);
  for (uint32_t t = 0; t < n_api; ++t) {
    acc_before[t] = (uint32_t)c->acc_ts.size();
    const uint8_t k = c->kinds[t];
    if (k != DRGPUM_API_ALLOC && k != DRGPUM_API_FREE) {
      c->acc_rank[t] = (uint32_t)c->acc_ts.size();
      c->acc_ts.push_back(t);
      c->acc_cs.push_back(k == DRGPUM_API_MEMCPY || k == DRGPUM_API_MEMSET);
    }
  }
  acc_before[n_api] = (uint32_t)c->acc_ts.size();
  c->n_acc = (uint32_t)c->acc_ts.size();

  // segment index: elementary segments between consecutive object boundaries
  std::vector<uint64_t>& pts = c->seg_start;
  pts.clear();
  pts.reserve(2 * n);
  for (const auto& o : c->objs) { pts.push_back(o.base); pts.push_back(o.base + o.size); }
  std::sort(pts.begin(), pts.end());
  pts.erase(std::unique(pts.begin(), pts.end()), pts.end());
  const uint64_t S = pts.size();
  if (S >= 0xFFFFFFFFull) return fail(c, DRGPUM_ENOMEM, "too many segments (%llu)", (unsigned long long)S);
  auto seg_of = [&](uint64_t a) { return (uint64_t)(std::lower_bound(pts.begin(), pts.end(), a) - pts.begin()); };
  std::vector<uint64_t> j0(n), j1(n);
  std::vector<uint64_t> cnt(S + 1, 0);
  uint64_t total = 0;
  for (uint64_t i = 0; i < n; ++i) {
    j0[i] = seg_of(c->objs[i].base);
    j1[i] = seg_of(c->objs[i].base + c->objs[i].size);
    total += j1[i] - j0[i];
    if (total >= 0xFFFFFFFFull)
      return fail(c, DRGPUM_ENOMEM, "segment index exceeds 2^32 candidate entries (address reuse depth)");
  }
  // candidate counts by a difference array, offsets by prefix sum
  std::vector<int64_t> diff(S + 1, 0);
  for (uint64_t i = 0; i < n; ++i) { diff[j0[i]]++; diff[j1[i]]--; }
  c->seg_cand_off.assign(S + 1, 0);
  int64_t run = 0;
  for (uint64_t j = 0; j < S; ++j) {
    run += diff[j];
    c->seg_cand_off[j + 1] = c->seg_cand_off[j] + (uint32_t)run;
  }
  c->cand.assign(total, CandEntry{0, 0});
  std::vector<uint32_t> fillp(c->seg_cand_off.begin(), c->seg_cand_off.end() - 1);
  std::vector<uint64_t> by_alloc(n);
  std::iota(by_alloc.begin(), by_alloc.end(), 0);
  std::stable_sort(by_alloc.begin(), by_alloc.end(), [&](uint64_t a, uint64_t b) {
    return c->objs[a].t_alloc < c->objs[b].t_alloc;
  });
  for (uint64_t i : by_alloc)
    for (uint64_t j = j0[i]; j < j1[i]; ++j) c->cand[fillp[j]++] = CandEntry{(uint32_t)i, c->objs[i].t_alloc};
  // R5: within a segment, consecutive candidates (by t_alloc) must have
  // disjoint open lifetimes: t_alloc(next) >= t_free(prev)
  for (uint64_t j = 0; j < S; ++j) {
    for (uint32_t k = c->seg_cand_off[j] + 1; k < c->seg_cand_off[j + 1]; ++k) {
      const auto& pv = c->objs[c->cand[k - 1].obj];
      const auto& nx = c->objs[c->cand[k].obj];
      if (nx.t_alloc < pv.t_free)
        return fail(c, DRGPUM_EOVERLAP, "objects %u and %u overlap in address and lifetime",
                    c->cand[k - 1].obj, c->cand[k].obj);
    }
  }
  if (n >= kMultiBit || total >= kMultiBit)
    return fail(c, DRGPUM_ENOMEM, "segment index needs < 2^31 objects and candidate entries");
  c->seg.assign(S, SegEntry{0, kNone, 0});
  for (uint64_t j = 0; j < S; ++j) {
    SegEntry& e = c->seg[j];
    e.start = pts[j];
    const uint32_t c0 = c->seg_cand_off[j], k = c->seg_cand_off[j + 1] - c0;
    if (k == 1) { e.ref = c->cand[c0].obj; e.aux = c->cand[c0].t_alloc; }
    else if (k > 1) { e.ref = kMultiBit | c0; e.aux = k; }
  }
  // level-1 keys for shared memory
  c->l1_stride = (uint32_t)std::max<uint64_t>(1, (S + kL1MaxKeys - 1) / kL1MaxKeys);
  c->l1.clear();
  for (uint64_t j = 0; j < S; j += c->l1_stride) c->l1.push_back(pts[j]);

  // shadow layout: bitmaps (each 4-word aligned) then hit rows
  c->layout.assign(n, drgpum_object_layout_t{});
  c->dobj.assign(n, DevObj{});
  c->n_hit.assign(n, 0);
  c->tiles.clear();
  c->tile_off.assign(n + 1, 0);
  uint64_t bw = 0;
  for (uint64_t i = 0; i < n; ++i) {
    const auto& o = c->objs[i];
    const uint64_t ne = o.size / o.elem_size;
    const uint64_t words = (ne + 31) / 32;
    c->layout[i].bitmap_word = bw;
    c->tile_off[i] = (uint32_t)c->tiles.size();
    for (uint64_t w = 0; w < words; w += kTileWords) {
      Tile t;
      t.word_lo = bw + w;
      t.n_words = (uint32_t)std::min<uint64_t>(kTileWords, words - w);
      t.obj = (uint32_t)i;
      t.elem_lo = w * 32;
      t.n_bits = std::min<uint64_t>(ne - w * 32, uint64_t(kTileWords) * 32);
      c->tiles.push_back(t);
    }
    bw += align_up(words, 4);
  }
  if (c->tiles.size() >= 0xFFFFFFFFull) return fail(c, DRGPUM_ENOMEM, "too many reduction tiles");
  c->n_small_tiles = 0;
  for (const Tile& t : c->tiles) c->n_small_tiles += t.n_words <= 128;
  c->tile_off[n] = (uint32_t)c->tiles.size();
  c->groups.clear();
  c->group_off.assign(n + 1, 0);
  c->small_prefix.clear();
  for (uint64_t i = 0; i < n; ++i) {
    c->group_off[i] = (uint32_t)c->groups.size();
    for (uint32_t t = c->tile_off[i]; t < c->tile_off[i + 1]; t += kGroupTiles)
      c->groups.push_back(Group{t, std::min<uint32_t>(kGroupTiles, c->tile_off[i + 1] - t)});
  }
  c->group_off[n] = (uint32_t)c->groups.size();
  c->bitmap_words = bw;
  uint64_t hw = 0;
  for (uint64_t i = 0; i < n; ++i) {
    const auto& o = c->objs[i];
    const uint32_t r_lo = acc_before[o.t_alloc];
    const uint32_t r_hi = o.t_free == DRGPUM_NEVER ? c->n_acc : acc_before[o.t_free];
    c->layout[i].r_lo = r_lo;
    c->layout[i].n_hit_apis = r_hi - r_lo;
    c->layout[i].hit_word = hw;
    c->n_hit[i] = r_hi - r_lo;
    DevObj d;
    d.base = o.base;
    d.end = o.base + o.size;
    d.bm_bit = c->layout[i].bitmap_word * 32;
    d.hit_word = bw + hw;
    d.t_alloc = o.t_alloc;
    d.t_free = o.t_free;
    d.r_lo = r_lo;
    d.shift = ilog2(o.elem_size);
    c->dobj[i] = d;
    hw += (2ull * (r_hi - r_lo) + 31) / 32;
  }
  c->hit_words = hw;
  c->elem_base.assign(n, 0);
  uint64_t eb = 0;
  for (uint64_t i = 0; i < n; ++i) { c->elem_base[i] = eb; eb += c->objs[i].size / c->objs[i].elem_size; }
  c->n_elem_total = eb;
  c->fq_pos_bits = std::max<uint32_t>(1, bits_for(kFreqPosMul * eb));   // NEXT-2 keys: 4*element + type
  c->fq_digits = (c->fq_pos_bits + bits_for(c->n_acc) + kFreqRadixBits - 1) / kFreqRadixBits;   // radix passes
  c->slot_base.assign(n, 0);
  uint64_t sb = 0;
  for (uint64_t i = 0; i < n; ++i) { c->slot_base[i] = sb; sb += c->n_hit[i]; }
  c->n_slots = sb;

  return compute_layout(c);
}

// Workspace layout for the loaded program (and the enabled features).
drgpum_status compute_layout(drgpum_ctx* c) {
  const uint64_t n = c->n_obj;
  const uint32_t n_api = c->n_api;
  const uint64_t S = c->seg_start.size();
  const uint64_t total = c->cand.size();
  Layout& L = c->L;
  uint64_t off = 0;
  auto put = [&](uint64_t bytes) { uint64_t o = off; off = align_up(off + bytes); return o; };
  L.orw = put(4 * (c->bitmap_words + c->hit_words));
  L.first = put(4 * n);
  L.last = put(4 * n);
  L.ctr = put(8 * C_SLOTS);
  L.cons = put(8 * kMaxPeers);   // per-rank consistency counts after gather_peers
  L.rfull = put(4 * n);
  L.dyn_end = off;
  L.objs = put(sizeof(DevObj) * n);
  L.seg_start = put(8 * S);
  L.seg_cand_off = put(4 * (S + 1));
  L.seg = put(sizeof(SegEntry) * S);
  L.cand = put(sizeof(CandEntry) * total);
  L.l1 = put(8 * c->l1.size());
  L.acc_rank = put(4ull * n_api);
  L.acc_ts = put(4ull * c->n_acc);
  L.acc_cs = put(c->n_acc);
  L.n_hit = put(4 * n);
  L.tiles = put(sizeof(Tile) * c->tiles.size());
  L.pmask = put(8 * n);                      // owned merge: peers that touched each object
  L.tile_part = put(sizeof(BitMonoid) * c->tiles.size());
  L.groups = put(sizeof(Group) * c->groups.size());
  L.group_off = put(4 * (n + 1));
  L.group_part = put(sizeof(BitMonoid) * c->groups.size());
  L.stats = put(sizeof(drgpum_object_stats_t) * n);
  L.reports = put(sizeof(drgpum_pattern_report_t) * n);
  L.rq = put(sizeof(RangeEntry) * c->rq_cap);
  L.hints = put(sizeof(ChunkHint) * kHintCap);
  L.stage = put(2 * kStageRecords * sizeof(drgpum_record_t));
  L.sa_owner = L.sa_overlap = L.sa_elem_base = L.sa_q = L.sa_qcount = L.sa_end = L.sa_group = off;
  if (c->features & (DRGPUM_FEATURE_STRUCTURED | DRGPUM_FEATURE_FREQUENCY)) {
    L.sa_elem_base = put(8 * n);              // shared by both features
    L.sa_group = put(n_api);                  // API group of the SA pass [R23] (1 = in)
  }
  if (c->features & DRGPUM_FEATURE_STRUCTURED) {
    L.sa_owner = put(4 * c->n_elem_total);
    L.sa_overlap = put(4 * n);
    L.sa_qcount = put(8);
    L.sa_end = off;                           // [sa_owner, sa_end) is zeroed per trace
    L.sa_q = put(sizeof(SaRange) * c->sa_q_cap);
  }
  L.fq_acc = L.fq_state = L.fq_ctl = L.fq_end = L.fq_acc_q = L.fq_slot_base = off;
  L.fq_out_count = L.fq_out_first = L.fq_keys0 = L.fq_keys1 = L.fq_hist = L.fq_offs = L.fq_part = off;
  if (c->features & DRGPUM_FEATURE_FREQUENCY) {
    L.fq_acc = put(24 * c->n_slots);
    L.fq_state = put(16);
    L.fq_ctl = put(8 * kFreqCtlWords);
    L.fq_end = off;                           // [fq_acc, fq_end) is zeroed per trace
    L.fq_acc_q = put(24 * c->n_slots);
    L.fq_slot_base = put(8 * n);
    L.fq_out_count = put(4 * n);
    L.fq_out_first = put(4 * n);
    L.fq_keys0 = put(8 * freq_cap(c));
    L.fq_keys1 = put(8 * freq_cap(c));
    L.fq_hist = put(4ull * (1u << kFreqRadixBits) * freq_max_tiles(c));
    L.fq_offs = put(4ull * (1u << kFreqRadixBits) * freq_max_tiles(c));
    L.fq_part = put(4 * (4 * freq_max_tiles(c) + 64));
  }
  L.total = off;
  return DRGPUM_OK;
}

drgpum_status validate(drgpum_ctx* c, const drgpum_object_t* objs, uint64_t n_obj,
                       const uint8_t* kinds, uint32_t n_api) {
  if (n_api >= 0x80000000u) return fail(c, DRGPUM_EINVAL, "n_api >= 2^31");
  if (n_obj >= 0xFFFFFFFFull) return fail(c, DRGPUM_EINVAL, "n_obj >= 2^32-1");
  if (n_api && !kinds) return fail(c, DRGPUM_EINVAL, "api kinds is NULL");
  if (n_obj && !objs) return fail(c, DRGPUM_EINVAL, "objects is NULL");
  for (uint32_t t = 0; t < n_api; ++t)
    if (kinds[t] > DRGPUM_API_KERNEL) return fail(c, DRGPUM_EINVAL, "api %u has kind %u", t, kinds[t]);
  for (uint64_t i = 0; i < n_obj; ++i) {
    const drgpum_object_t& o = objs[i];
    const uint32_t E = o.elem_size;
    const char* why = nullptr;
    if (o.size == 0) why = "size 0";
    else if (!(E == 1 || E == 2 || E == 4 || E == 8 || E == 16)) why = "elem_size not in {1,2,4,8,16}";
    else if (o.size % E) why = "size not a multiple of elem_size";
    else if (o.base > UINT64_MAX - o.size) why = "base+size overflows";
    else if (o.t_alloc >= n_api || kinds[o.t_alloc] != DRGPUM_API_ALLOC) why = "t_alloc is not an ALLOC API";
    else if (o.t_free != DRGPUM_NEVER &&
             (o.t_free >= n_api || o.t_free <= o.t_alloc || kinds[o.t_free] != DRGPUM_API_FREE))
      why = "t_free is not a FREE API after t_alloc";
    if (why) return fail(c, DRGPUM_EINVAL, "object %llu: %s", (unsigned long long)i, why);
  }
  return DRGPUM_OK;
}

#ifndef DRGPUM_SPARSE_RESET
#define DRGPUM_SPARSE_RESET 1
#endif
#ifndef DRGPUM_SPARSE_MERGE
#define DRGPUM_SPARSE_MERGE 1   // owned merge reads only the peers that touched an object
#endif
drgpum_status enqueue_reset(drgpum_ctx* ctx, cudaStream_t s, bool dense) {
  // dynamic state: shadow words, last, counters = 0; first = NEVER.  Dense
  // (bind: the memory is fresh): one pass over all of it.  Sparse (every
  // later reset): only the touched objects' bitmap tiles and hit rows -- the
  // OR words of an object are nonzero only if its first[] is not NEVER --,
  // then the small sections from first[] on.
  const bool consumed = ctx->consumed;   // bitmaps already zeroed by a consuming finalize
  ctx->consumed = false;
  if (dense || !DRGPUM_SPARSE_RESET) {
    ctx->launches += launch_reset(ctx->ws, ctx->L.dyn_end, ctx->L.first, 4 * ctx->n_obj, ctx->num_sms, s);
  } else {
    ctx->launches += launch_reset_touched(at<uint32_t>(ctx, ctx->L.orw), at<Tile>(ctx, ctx->L.tiles),
                                          consumed ? 0 :
                                          ctx->tiles.size(), at<DevObj>(ctx, ctx->L.objs),
                                          at<uint32_t>(ctx, ctx->L.n_hit), at<uint32_t>(ctx, ctx->L.first),
                                          ctx->n_obj, 2 * ctx->n_small_tiles > ctx->tiles.size(),
                                          ctx->num_sms, s);
    ctx->launches += launch_reset(ctx->ws + ctx->L.first, ctx->L.dyn_end - ctx->L.first, 0, 4 * ctx->n_obj,
                                  ctx->num_sms, s);
  }
  if (ctx->features & DRGPUM_FEATURE_STRUCTURED)
    CK(cudaMemsetAsync(ctx->ws + ctx->L.sa_owner, 0, ctx->L.sa_end - ctx->L.sa_owner, s));
  if (ctx->features & DRGPUM_FEATURE_FREQUENCY)
    CK(cudaMemsetAsync(ctx->ws + ctx->L.fq_acc, 0, ctx->L.fq_end - ctx->L.fq_acc, s));
  ctx->final_valid = false;
  ctx->owned = ctx->gathered = false;
  return DRGPUM_OK;
}

AttrParams attr_params(drgpum_ctx* c, const drgpum_record_t* recs, uint64_t n) {
  AttrParams p;
  p.recs = reinterpret_cast<const uint4*>(recs);
  p.n = n;
  p.objs = at<DevObj>(c, c->L.objs);
  p.seg_start = at<uint64_t>(c, c->L.seg_start);
  p.seg_cand_off = at<uint32_t>(c, c->L.seg_cand_off);
  p.seg = at<SegEntry>(c, c->L.seg);
  p.cand = at<CandEntry>(c, c->L.cand);
  p.l1 = at<uint64_t>(c, c->L.l1);
  p.n_seg = (uint32_t)c->seg_start.size();
  p.n_l1 = (uint32_t)c->l1.size();
  p.l1_stride = c->l1_stride;
  p.n_api = c->n_api;
  p.acc_rank = at<uint32_t>(c, c->L.acc_rank);
  p.orw = at<uint32_t>(c, c->L.orw);
  p.first = at<uint32_t>(c, c->L.first);
  p.last = at<uint32_t>(c, c->L.last);
  p.ctr = at<unsigned long long>(c, c->L.ctr);
  p.rfull = at<uint32_t>(c, c->L.rfull);
  p.rq = at<RangeEntry>(c, c->L.rq);
  p.rq_cap = c->rq_cap;
  p.hints = at<ChunkHint>(c, c->L.hints);
  p.hint_cap = kHintCap;
  p.rq_slot = (c->attr_calls & 1) ? C_RQ_COUNT_ALT : C_RQ_COUNT;
  p.chunk_shift = 13;   // launch_attribute sets the attribution's own
  // work chunks may grow to 32768 records when most bitmap tiles are small
  // (objects of <= 4096 elements: the per-warp scratch path, C5); A/B in
  // DESIGN.md section 6 (C5 / C4 faster with larger chunks, C3 slower)
  p.chunk_max_shift = 2 * c->n_small_tiles > c->tiles.size() ? kChunkMaxShiftSmall : 13;
  return p;
}

FreqParams fq_params(drgpum_ctx* c, const drgpum_record_t* recs, uint64_t n) {
  FreqParams q;
  q.a = attr_params(c, recs, n);
  q.elem_base = at<uint64_t>(c, c->L.sa_elem_base);
  q.slot_base = at<uint64_t>(c, c->L.fq_slot_base);
  q.acc = at<unsigned long long>(c, c->L.fq_acc);
  q.acc_q = at<unsigned long long>(c, c->L.fq_acc_q);
  q.state = at<uint32_t>(c, c->L.fq_state);
  q.ctl = at<unsigned long long>(c, c->L.fq_ctl);
  q.keys0 = at<uint64_t>(c, c->L.fq_keys0);
  q.keys1 = at<uint64_t>(c, c->L.fq_keys1);
  q.cap = freq_cap(c);
  q.hist = at<uint32_t>(c, c->L.fq_hist);
  q.offs = at<uint32_t>(c, c->L.fq_offs);
  q.part = at<uint32_t>(c, c->L.fq_part);
  q.max_tiles = freq_max_tiles(c);
  q.n_obj = c->n_obj;
  q.pos_bits = c->fq_pos_bits;
  q.n_digits = c->fq_digits;
  return q;
}

// the NEXT-2 pass over n device records, in sub-calls of at most fq_recs
int launch_frequency_calls(drgpum_ctx* c, const drgpum_record_t* recs, uint64_t n, cudaStream_t s) {
  int launches = 0;
  for (uint64_t i = 0; i < n; i += c->fq_recs)
    launches += launch_frequency(fq_params(c, recs + i, std::min(c->fq_recs, n - i)), c->num_sms, s);
  return launches;
}

SaParams sa_params(drgpum_ctx* c, const drgpum_record_t* recs, uint64_t n) {
  SaParams q;
  q.a = attr_params(c, recs, n);
  q.owner = at<uint32_t>(c, c->L.sa_owner);
  q.elem_base = at<uint64_t>(c, c->L.sa_elem_base);
  q.overlap = at<uint32_t>(c, c->L.sa_overlap);
  q.q = at<SaRange>(c, c->L.sa_q);
  q.q_cap = c->sa_q_cap;
  q.q_count = at<unsigned long long>(c, c->L.sa_qcount);
  q.in_group = at<uint8_t>(c, c->L.sa_group);
  return q;
}

}  // namespace

extern "C" {

DRGPUM_API drgpum_status drgpum_create(int cuda_device, drgpum_ctx** out) {
  if (!out) return DRGPUM_EINVAL;
  *out = nullptr;
  drgpum_ctx* ctx = new drgpum_ctx();
  ctx->device = cuda_device;
  drgpum_status s = set_device(ctx);
  if (s != DRGPUM_OK) { *out = ctx; return s; }
  cudaDeviceGetAttribute(&ctx->num_sms, cudaDevAttrMultiProcessorCount, cuda_device);
  *out = ctx;
  return DRGPUM_OK;
}

DRGPUM_API drgpum_status drgpum_objects_load(drgpum_ctx* ctx, const drgpum_object_t* h_objs,
                                             uint64_t n_obj, const uint8_t* h_api_kinds,
                                             uint32_t n_api) {
  if (!ctx) return DRGPUM_EINVAL;
  drgpum_status s = validate(ctx, h_objs, n_obj, h_api_kinds, n_api);
  if (s != DRGPUM_OK) return s;
  drgpum_ctx tmp;  // build into a scratch context so a failure leaves ctx unchanged
  tmp.n_obj = n_obj;
  tmp.n_api = n_api;
  tmp.objs.assign(h_objs, h_objs + n_obj);
  tmp.kinds.assign(h_api_kinds, h_api_kinds + n_api);
  tmp.rq_cap = ctx->rq_cap;
  tmp.sa_q_cap = ctx->sa_q_cap;
  tmp.fq_recs = ctx->fq_recs;
  s = build_tables(&tmp);
  if (s != DRGPUM_OK) { ctx->err = tmp.err; return s; }
  ctx->n_obj = tmp.n_obj; ctx->n_api = tmp.n_api; ctx->n_acc = tmp.n_acc;
  ctx->objs.swap(tmp.objs); ctx->kinds.swap(tmp.kinds); ctx->dobj.swap(tmp.dobj);
  ctx->seg_start.swap(tmp.seg_start); ctx->seg_cand_off.swap(tmp.seg_cand_off); ctx->seg.swap(tmp.seg);
  ctx->cand.swap(tmp.cand); ctx->l1.swap(tmp.l1); ctx->l1_stride = tmp.l1_stride;
  ctx->acc_rank.swap(tmp.acc_rank); ctx->acc_ts.swap(tmp.acc_ts); ctx->acc_cs.swap(tmp.acc_cs);
  ctx->n_hit.swap(tmp.n_hit); ctx->tiles.swap(tmp.tiles); ctx->tile_off.swap(tmp.tile_off);
  ctx->groups.swap(tmp.groups); ctx->group_off.swap(tmp.group_off); ctx->small_prefix.clear();
  ctx->n_small_tiles = tmp.n_small_tiles;
  ctx->elem_base.swap(tmp.elem_base); ctx->n_elem_total = tmp.n_elem_total;
  ctx->slot_base.swap(tmp.slot_base); ctx->n_slots = tmp.n_slots;
  ctx->fq_pos_bits = tmp.fq_pos_bits; ctx->fq_digits = tmp.fq_digits;
  ctx->features = 0;
  ctx->layout.swap(tmp.layout);
  ctx->bitmap_words = tmp.bitmap_words; ctx->hit_words = tmp.hit_words;
  ctx->L = tmp.L;
  ctx->ws = nullptr;
  ctx->ws_bytes = 0;
  ctx->state = S_LOADED;
  ctx->final_valid = false;
  return DRGPUM_OK;
}

DRGPUM_API drgpum_status drgpum_set_finalize_consume(drgpum_ctx* ctx, int on) {
  if (!ctx) return DRGPUM_EINVAL;
  ctx->fin_consume = on != 0;
  return DRGPUM_OK;
}

DRGPUM_API drgpum_status drgpum_set_features(drgpum_ctx* ctx, uint32_t features) {
  if (!ctx) return DRGPUM_EINVAL;
  if (ctx->state != S_LOADED) return fail(ctx, DRGPUM_ESTATE, "set_features must follow objects_load and precede workspace_bind");
  if (features & ~uint32_t(DRGPUM_FEATURE_STRUCTURED | DRGPUM_FEATURE_FREQUENCY))
    return fail(ctx, DRGPUM_EINVAL, "unknown feature bits");
  ctx->features = features;
  drgpum_status r = compute_layout(ctx);
  if (r == DRGPUM_OK && (features & DRGPUM_FEATURE_FREQUENCY) && ctx->fq_pos_bits + bits_for(ctx->n_acc) > 64)
    return fail(ctx, DRGPUM_EINVAL, "frequency analysis: (API rank, 2 x element) keys exceed 64 bits");
  return r;
}

DRGPUM_API drgpum_status drgpum_set_queue_capacity(drgpum_ctx* ctx, uint32_t range_entries,
                                                   uint32_t aux_entries) {
  if (!ctx) return DRGPUM_EINVAL;
  if (ctx->state != S_LOADED)
    return fail(ctx, DRGPUM_ESTATE, "set_queue_capacity must follow objects_load and precede workspace_bind");
  if (range_entries > (1u << 24) || aux_entries > (1u << 24))
    return fail(ctx, DRGPUM_EINVAL, "queue capacity above 2^24 entries");
  if (range_entries) ctx->rq_cap = range_entries;
  if (aux_entries) ctx->sa_q_cap = aux_entries;
  return compute_layout(ctx);
}

DRGPUM_API drgpum_status drgpum_set_frequency_capacity(drgpum_ctx* ctx, uint64_t records_per_call) {
  if (!ctx) return DRGPUM_EINVAL;
  if (ctx->state != S_LOADED)
    return fail(ctx, DRGPUM_ESTATE, "set_frequency_capacity must follow objects_load and precede workspace_bind");
  if (records_per_call < 1024 || records_per_call > (1ull << 31))
    return fail(ctx, DRGPUM_EINVAL, "records_per_call outside [1024, 2^31]");
  ctx->fq_recs = records_per_call;
  return compute_layout(ctx);
}

DRGPUM_API drgpum_status drgpum_structured(drgpum_ctx* ctx, uint8_t* h_sa, uint8_t* h_overlap, void* stream) {
  if (!ctx) return DRGPUM_EINVAL;
  if (ctx->state < S_BOUND) return fail(ctx, DRGPUM_ESTATE, "structured before workspace_bind");
  if (drgpum_status _d = set_device(ctx)) return _d;
  if (!(ctx->features & DRGPUM_FEATURE_STRUCTURED))
    return fail(ctx, DRGPUM_ESTATE, "DRGPUM_FEATURE_STRUCTURED was not enabled");
  cudaStream_t strm = as_stream(stream);
  // accessing APIs of the group per object [R23]: the finalized n_access_apis
  // when the group is every API, else counted on the hit rows
  std::vector<uint64_t> n_in(ctx->n_obj, 0);
  const bool all = std::all_of(ctx->api_group.begin(), ctx->api_group.end(), [](uint8_t g) { return g != 0; });
  if (all) {
    std::vector<drgpum_object_stats_t> st(ctx->n_obj);
    drgpum_status s = drgpum_object_stats(ctx, st.data(), nullptr, stream);
    if (s != DRGPUM_OK) return s;
    for (uint64_t o = 0; o < ctx->n_obj; ++o) n_in[o] = st[o].n_access_apis;
  } else {
    std::vector<uint64_t> off;
    std::vector<uint32_t> api;
    std::vector<uint8_t> rw;
    drgpum_status s = gather_accesses(ctx, strm, off, api, rw);
    if (s != DRGPUM_OK) return s;
    for (uint64_t o = 0; o < ctx->n_obj; ++o)
      for (uint64_t k = off[o]; k < off[o + 1]; ++k) n_in[o] += ctx->api_group[api[k]] ? 1 : 0;
  }
  std::vector<uint32_t> ov(ctx->n_obj);
  if (ctx->n_obj) {
    CK(cudaMemcpyAsync(ov.data(), ctx->ws + ctx->L.sa_overlap, 4 * ctx->n_obj, cudaMemcpyDeviceToHost, strm));
    CK(cudaStreamSynchronize(strm));
  }
  for (uint64_t o = 0; o < ctx->n_obj; ++o) {
    if (h_overlap) h_overlap[o] = ov[o] ? 1 : 0;
    if (h_sa) h_sa[o] = (n_in[o] >= 2 && !ov[o]) ? 1 : 0;
  }
  return DRGPUM_OK;
}

DRGPUM_API drgpum_status drgpum_set_api_group(drgpum_ctx* ctx, const uint8_t* h_in_group, void* stream) {
  if (!ctx) return DRGPUM_EINVAL;
  if (ctx->state < S_BOUND) return fail(ctx, DRGPUM_ESTATE, "set_api_group before workspace_bind");
  if (drgpum_status _d = set_device(ctx)) return _d;
  if (!(ctx->features & (DRGPUM_FEATURE_STRUCTURED | DRGPUM_FEATURE_FREQUENCY)))
    return fail(ctx, DRGPUM_ESTATE, "set_api_group needs DRGPUM_FEATURE_STRUCTURED or _FREQUENCY");
  for (uint32_t t = 0; t < ctx->n_api; ++t) ctx->api_group[t] = h_in_group ? (h_in_group[t] ? 1 : 0) : 1;
  cudaStream_t st = as_stream(stream);
  if (ctx->n_api) {
    CK(cudaMemcpyAsync(ctx->ws + ctx->L.sa_group, ctx->api_group.data(), ctx->n_api, cudaMemcpyHostToDevice, st));
    CK(cudaStreamSynchronize(st));   // the host copy may change with the next call
  }
  return DRGPUM_OK;
}

static drgpum_status frequency_ready(drgpum_ctx* ctx, cudaStream_t st) {
  if (ctx->state < S_BOUND) return fail(ctx, DRGPUM_ESTATE, "frequency before workspace_bind");
  if (drgpum_status _d = set_device(ctx)) return _d;
  if (!(ctx->features & DRGPUM_FEATURE_FREQUENCY))
    return fail(ctx, DRGPUM_ESTATE, "DRGPUM_FEATURE_FREQUENCY was not enabled");
  uint32_t state[2];
  CK(cudaMemcpyAsync(state, ctx->ws + ctx->L.fq_state, 8, cudaMemcpyDeviceToHost, st));
  CK(cudaStreamSynchronize(st));
  if (state[0] & 1) return fail(ctx, DRGPUM_EINVAL, "frequency analysis needs records in API (timestamp) order");
  if (state[0]) return fail(ctx, DRGPUM_ENOMEM, "frequency analysis: one API's events exceed the key capacity "
                            "(drgpum_set_frequency_capacity)");
  // the sums including the API carried at the end of the last call
  ctx->launches += launch_frequency_query(fq_params(ctx, nullptr, 0), ctx->n_slots, ctx->num_sms, st);
  CK(cudaGetLastError());
  return DRGPUM_OK;
}

DRGPUM_API drgpum_status drgpum_frequency(drgpum_ctx* ctx, uint32_t pct, uint32_t* h_count,
                                          uint32_t* h_first, void* stream) {
  if (!ctx) return DRGPUM_EINVAL;
  cudaStream_t st = as_stream(stream);
  drgpum_status r = frequency_ready(ctx, st);
  if (r != DRGPUM_OK) return r;
  FreqReduceParams q;
  q.acc = at<unsigned long long>(ctx, ctx->L.fq_acc_q);
  q.slot_base = at<uint64_t>(ctx, ctx->L.fq_slot_base);
  q.n_hit = at<uint32_t>(ctx, ctx->L.n_hit);
  q.objs = at<DevObj>(ctx, ctx->L.objs);
  q.acc_ts = at<uint32_t>(ctx, ctx->L.acc_ts);
  q.n_obj = ctx->n_obj;
  q.pct = pct;
  q.out_count = at<uint32_t>(ctx, ctx->L.fq_out_count);
  q.out_first = at<uint32_t>(ctx, ctx->L.fq_out_first);
  ctx->launches += launch_frequency_reduce(q, ctx->num_sms, st);
  CK(cudaGetLastError());
  if (h_count && ctx->n_obj)
    CK(cudaMemcpyAsync(h_count, q.out_count, 4 * ctx->n_obj, cudaMemcpyDeviceToHost, st));
  if (h_first && ctx->n_obj)
    CK(cudaMemcpyAsync(h_first, q.out_first, 4 * ctx->n_obj, cudaMemcpyDeviceToHost, st));
  CK(cudaStreamSynchronize(st));
  return DRGPUM_OK;
}

DRGPUM_API drgpum_status drgpum_frequency_slots(drgpum_ctx* ctx, uint64_t* h_acc, uint64_t* n_slots,
                                                void* stream) {
  if (!ctx || !n_slots) return DRGPUM_EINVAL;
  cudaStream_t st = as_stream(stream);
  drgpum_status r = frequency_ready(ctx, st);
  if (r != DRGPUM_OK) return r;
  *n_slots = ctx->n_slots;
  if (h_acc && ctx->n_slots) {
    CK(cudaMemcpyAsync(h_acc, ctx->ws + ctx->L.fq_acc_q, 24 * ctx->n_slots, cudaMemcpyDeviceToHost, st));
    CK(cudaStreamSynchronize(st));
  }
  return DRGPUM_OK;
}

DRGPUM_API drgpum_status drgpum_slice_frequency(drgpum_ctx* ctx, uint32_t pct, uint8_t* h_match,
                                                uint64_t* h_moments, void* stream) {
  if (!ctx) return DRGPUM_EINVAL;
  cudaStream_t st = as_stream(stream);
  drgpum_status r = frequency_ready(ctx, st);
  if (r != DRGPUM_OK) return r;
  std::vector<uint64_t> acc(3 * ctx->n_slots);
  if (ctx->n_slots) {
    CK(cudaMemcpyAsync(acc.data(), ctx->ws + ctx->L.fq_acc_q, 24 * ctx->n_slots, cudaMemcpyDeviceToHost, st));
    CK(cudaStreamSynchronize(st));
  }
  // [R22b] per object: over the group's accessing APIs A, F_A = S1 of slot
  // (O, A); CV of {F_A} > pct% iff (n*S2 - S1^2) * 100^2 > pct^2 * S1^2
  uint64_t slot = 0;
  for (uint64_t o = 0; o < ctx->n_obj; ++o) {
    const auto& l = ctx->layout[o];
    uint64_t n = 0, s1 = 0;
    unsigned __int128 s2 = 0;
    for (uint32_t k = 0; k < l.n_hit_apis; ++k, ++slot) {
      const uint64_t F = acc[3 * slot + 1];
      if (!acc[3 * slot] || !ctx->api_group[ctx->acc_ts[l.r_lo + k]]) continue;
      ++n;
      s1 += F;
      s2 += (unsigned __int128)F * F;
    }
    const unsigned __int128 S1 = s1, var = (unsigned __int128)n * s2 - S1 * S1;
    if (h_match) h_match[o] = (s1 > 0 && var * 10000 > (unsigned __int128)pct * pct * S1 * S1) ? 1 : 0;
    if (h_moments) {
      h_moments[4 * o] = n;
      h_moments[4 * o + 1] = s1;
      h_moments[4 * o + 2] = (uint64_t)s2;
      h_moments[4 * o + 3] = (uint64_t)(s2 >> 64);
    }
  }
  return DRGPUM_OK;
}

DRGPUM_API drgpum_status drgpum_workspace_size(const drgpum_ctx* ctx, uint64_t* bytes) {
  if (!ctx || !bytes) return DRGPUM_EINVAL;
  if (ctx->state < S_LOADED) return DRGPUM_ESTATE;
  *bytes = ctx->L.total;
  return DRGPUM_OK;
}

DRGPUM_API drgpum_status drgpum_workspace_bind(drgpum_ctx* ctx, void* d_ws, uint64_t bytes, void* stream) {
  if (!ctx) return DRGPUM_EINVAL;
  if (ctx->state < S_LOADED) return fail(ctx, DRGPUM_ESTATE, "workspace_bind before objects_load");
  if (!d_ws || (reinterpret_cast<uintptr_t>(d_ws) % kAlign))
    return fail(ctx, DRGPUM_EINVAL, "workspace must be non-NULL and 256-B aligned");
  if (bytes < ctx->L.total)
    return fail(ctx, DRGPUM_ENOMEM, "workspace has %llu bytes, needs %llu",
                (unsigned long long)bytes, (unsigned long long)ctx->L.total);
  drgpum_status s = set_device(ctx);
  if (s != DRGPUM_OK) return s;
  // per-device kernel attributes and occupancy, kept in the context
  ctx->attr_occ = attribute_occupancy();
  CK(cudaGetLastError());
  cudaStream_t st = as_stream(stream);
  ctx->ws = static_cast<uint8_t*>(d_ws);
  ctx->ws_bytes = bytes;
  const Layout& L = ctx->L;
  auto up = [&](uint64_t off, const void* src, uint64_t n) -> drgpum_status {
    if (!n) return DRGPUM_OK;
    CK(cudaMemcpyAsync(ctx->ws + off, src, n, cudaMemcpyHostToDevice, st));
    return DRGPUM_OK;
  };
  const uint64_t n = ctx->n_obj;
  drgpum_status r;
  if ((r = up(L.objs, ctx->dobj.data(), sizeof(DevObj) * n))) return r;
  if ((r = up(L.seg_start, ctx->seg_start.data(), 8 * ctx->seg_start.size()))) return r;
  if ((r = up(L.seg_cand_off, ctx->seg_cand_off.data(), 4 * ctx->seg_cand_off.size()))) return r;
  if ((r = up(L.seg, ctx->seg.data(), sizeof(SegEntry) * ctx->seg.size()))) return r;
  if ((r = up(L.cand, ctx->cand.data(), sizeof(CandEntry) * ctx->cand.size()))) return r;
  if ((r = up(L.l1, ctx->l1.data(), 8 * ctx->l1.size()))) return r;
  if ((r = up(L.acc_rank, ctx->acc_rank.data(), 4 * ctx->acc_rank.size()))) return r;
  if ((r = up(L.acc_ts, ctx->acc_ts.data(), 4 * ctx->acc_ts.size()))) return r;
  if ((r = up(L.acc_cs, ctx->acc_cs.data(), ctx->acc_cs.size()))) return r;
  if ((r = up(L.n_hit, ctx->n_hit.data(), 4 * n))) return r;
  if ((r = up(L.tiles, ctx->tiles.data(), sizeof(Tile) * ctx->tiles.size()))) return r;
  if ((r = up(L.groups, ctx->groups.data(), sizeof(Group) * ctx->groups.size()))) return r;
  if ((r = up(L.group_off, ctx->group_off.data(), 4 * ctx->group_off.size()))) return r;
  if (ctx->features & (DRGPUM_FEATURE_STRUCTURED | DRGPUM_FEATURE_FREQUENCY)) {
    if ((r = up(L.sa_elem_base, ctx->elem_base.data(), 8 * n))) return r;
    ctx->api_group.assign(ctx->n_api, 1);
    if ((r = up(L.sa_group, ctx->api_group.data(), ctx->n_api))) return r;
  }
  if (ctx->features & DRGPUM_FEATURE_FREQUENCY)
    if ((r = up(L.fq_slot_base, ctx->slot_base.data(), 8 * n))) return r;
  if ((r = enqueue_reset(ctx, st, true))) return r;
  // host vectors stay alive in ctx, so the async uploads are safe; make the
  // bind synchronous anyway so callers may immediately reuse their stream
  CK(cudaStreamSynchronize(st));
  ctx->state = S_BOUND;
  return DRGPUM_OK;
}

DRGPUM_API drgpum_status drgpum_reset(drgpum_ctx* ctx, void* stream) {
  if (!ctx) return DRGPUM_EINVAL;
  if (ctx->state < S_BOUND) return fail(ctx, DRGPUM_ESTATE, "reset before workspace_bind");
  if (drgpum_status _d = set_device(ctx)) return _d;
  return enqueue_reset(ctx, as_stream(stream), false);
}

DRGPUM_API drgpum_status drgpum_trace_attribute(drgpum_ctx* ctx, const drgpum_record_t* d_recs,
                                                uint64_t n, void* stream) {
  if (!ctx) return DRGPUM_EINVAL;
  if (ctx->state < S_BOUND) return fail(ctx, DRGPUM_ESTATE, "trace_attribute before workspace_bind");
  if (drgpum_status _d = set_device(ctx)) return _d;
  if (n == 0) return DRGPUM_OK;
  if (!d_recs || reinterpret_cast<uintptr_t>(d_recs) % 16)
    return fail(ctx, DRGPUM_EINVAL, "records must be non-NULL and 16-B aligned");
  if (ctx->consumed) return fail(ctx, DRGPUM_ESTATE, "trace_attribute after a consuming finalize: reset first");
  AttrParams p = attr_params(ctx, d_recs, n);
  ctx->launches += launch_attribute(p, ctx->num_sms, ctx->attr_occ, as_stream(stream));
  ctx->attr_calls++;
  if (ctx->features & DRGPUM_FEATURE_STRUCTURED)
    ctx->launches += launch_structured(sa_params(ctx, d_recs, n), ctx->num_sms, as_stream(stream));
  if (ctx->features & DRGPUM_FEATURE_FREQUENCY)
    ctx->launches += launch_frequency_calls(ctx, d_recs, n, as_stream(stream));
  ctx->final_valid = false;
  CK(cudaGetLastError());
  return DRGPUM_OK;
}

DRGPUM_API drgpum_status drgpum_trace_attribute_host(drgpum_ctx* ctx, const drgpum_record_t* h_recs,
                                                     uint64_t n, void* stream) {
  if (!ctx) return DRGPUM_EINVAL;
  if (ctx->state < S_BOUND) return fail(ctx, DRGPUM_ESTATE, "trace_attribute_host before workspace_bind");
  if (drgpum_status _d = set_device(ctx)) return _d;
  if (n == 0) return DRGPUM_OK;
  if (!h_recs) return fail(ctx, DRGPUM_EINVAL, "records is NULL");
  if (ctx->consumed) return fail(ctx, DRGPUM_ESTATE, "trace_attribute_host after a consuming finalize: reset first");
  cudaStream_t st = as_stream(stream);
  if (!ctx->copy_stream) {
    CK(cudaStreamCreateWithFlags(&ctx->copy_stream, cudaStreamNonBlocking));
    for (int i = 0; i < 2; ++i) {
      CK(cudaEventCreateWithFlags(&ctx->ev_copied[i], cudaEventDisableTiming));
      CK(cudaEventCreateWithFlags(&ctx->ev_used[i], cudaEventDisableTiming));
    }
  }
  drgpum_record_t* stage[2] = {at<drgpum_record_t>(ctx, ctx->L.stage),
                             at<drgpum_record_t>(ctx, ctx->L.stage) + kStageRecords};
  // the copy stream must not overwrite a stage before prior work on `st` is done with it
  CK(cudaEventRecord(ctx->ev_used[0], st));
  CK(cudaEventRecord(ctx->ev_used[1], st));
  uint64_t k = 0;
  for (uint64_t off = 0; off < n; off += kStageRecords, ++k) {
    const int b = int(k & 1);
    const uint64_t m = std::min<uint64_t>(kStageRecords, n - off);
    CK(cudaStreamWaitEvent(ctx->copy_stream, ctx->ev_used[b], 0));
    CK(cudaMemcpyAsync(stage[b], h_recs + off, m * sizeof(drgpum_record_t), cudaMemcpyHostToDevice,
                       ctx->copy_stream));
    CK(cudaEventRecord(ctx->ev_copied[b], ctx->copy_stream));
    CK(cudaStreamWaitEvent(st, ctx->ev_copied[b], 0));
    AttrParams p = attr_params(ctx, stage[b], m);
    ctx->launches += launch_attribute(p, ctx->num_sms, ctx->attr_occ, st);
    ctx->attr_calls++;
    if (ctx->features & DRGPUM_FEATURE_STRUCTURED)
      ctx->launches += launch_structured(sa_params(ctx, stage[b], m), ctx->num_sms, st);
    if (ctx->features & DRGPUM_FEATURE_FREQUENCY)
      ctx->launches += launch_frequency_calls(ctx, stage[b], m, st);
    CK(cudaEventRecord(ctx->ev_used[b], st));
  }
  CK(cudaStreamSynchronize(ctx->copy_stream));
  ctx->final_valid = false;
  CK(cudaGetLastError());
  return DRGPUM_OK;
}

DRGPUM_API drgpum_status drgpum_shadow_view(const drgpum_ctx* ctx, drgpum_shadow_view_t* out) {
  if (!ctx || !out) return DRGPUM_EINVAL;
  if (ctx->state < S_LOADED) return DRGPUM_ESTATE;
  out->or_off = ctx->L.orw;
  out->or_words = ctx->bitmap_words + ctx->hit_words;
  out->bitmap_words = ctx->bitmap_words;
  out->hit_words = ctx->hit_words;
  out->first_off = ctx->L.first;
  out->last_off = ctx->L.last;
  out->counters_off = ctx->L.ctr;
  out->n_obj = ctx->n_obj;
  return DRGPUM_OK;
}

DRGPUM_API drgpum_status drgpum_object_layout(const drgpum_ctx* ctx, drgpum_object_layout_t* h_out) {
  if (!ctx || (!h_out && ctx->n_obj)) return DRGPUM_EINVAL;
  if (ctx->state < S_LOADED) return DRGPUM_ESTATE;
  std::copy(ctx->layout.begin(), ctx->layout.end(), h_out);
  return DRGPUM_OK;
}

DRGPUM_API drgpum_status drgpum_merge_or(drgpum_ctx* ctx, const uint32_t* d_in, uint32_t n_src,
                                         uint64_t src_stride_words, uint64_t word_lo,
                                         uint64_t word_hi, void* stream) {
  if (!ctx) return DRGPUM_EINVAL;
  if (ctx->state < S_BOUND) return fail(ctx, DRGPUM_ESTATE, "merge_or before workspace_bind");
  if (ctx->consumed) return fail(ctx, DRGPUM_ESTATE, "merge_or after a consuming finalize: reset first");
  if (drgpum_status _d = set_device(ctx)) return _d;
  const uint64_t total = ctx->bitmap_words + ctx->hit_words;
  ctx->final_valid = false;  // the caller is merging state into this shadow
  if (word_lo > word_hi || word_hi > total)
    return fail(ctx, DRGPUM_EINVAL, "merge range [%llu,%llu) exceeds %llu words",
                (unsigned long long)word_lo, (unsigned long long)word_hi, (unsigned long long)total);
  if (word_hi == word_lo || n_src == 0) return DRGPUM_OK;
  if (!d_in) return fail(ctx, DRGPUM_EINVAL, "d_in is NULL");
  if (n_src > 1 && src_stride_words < word_hi - word_lo)
    return fail(ctx, DRGPUM_EINVAL, "src_stride_words smaller than the range");
  ctx->launches += launch_merge_or(at<uint32_t>(ctx, ctx->L.orw) + word_lo, d_in, n_src,
                                   src_stride_words, word_hi - word_lo, ctx->num_sms, as_stream(stream));
  ctx->final_valid = false;
  CK(cudaGetLastError());
  return DRGPUM_OK;
}

static drgpum_status check_peers(drgpum_ctx* ctx, const char* what, void* const* h_peer_ws,
                                 uint32_t n_peers, uint32_t rank, uint8_t** out) {
  if (!h_peer_ws || n_peers == 0 || n_peers > kMaxPeers || rank >= n_peers)
    return fail(ctx, DRGPUM_EINVAL, "%s: need 1 <= n_peers <= %u and rank < n_peers", what, kMaxPeers);
  if (h_peer_ws[rank] != ctx->ws)
    return fail(ctx, DRGPUM_EINVAL, "%s: h_peer_ws[rank] is not this context's workspace", what);
  for (uint32_t r = 0; r < n_peers; ++r) {
    if (!h_peer_ws[r] || reinterpret_cast<uintptr_t>(h_peer_ws[r]) % kAlign)
      return fail(ctx, DRGPUM_EINVAL, "%s: peer %u workspace NULL or not 256-B aligned", what, r);
    out[r] = static_cast<uint8_t*>(h_peer_ws[r]);
  }
  return DRGPUM_OK;
}

// Object boundary k of P: the first object o with bitmap_word(o) + o >= k/P of
// (bitmap words + objects) -- balances the merge (words) and the finalize
// (tiles + one warp per object).
static uint64_t owned_cut(const drgpum_ctx* c, uint32_t k, uint32_t P) {
  if (k == 0) return 0;
  if (k >= P) return c->n_obj;
  const uint64_t total = c->bitmap_words + c->n_obj;
  const uint64_t target = (uint64_t)((unsigned __int128)total * k / P);
  uint64_t lo = 0, hi = c->n_obj;   // f(n_obj) = total >= target
  while (lo < hi) {
    const uint64_t m = (lo + hi) / 2;
    if (c->layout[m].bitmap_word + m >= target) hi = m; else lo = m + 1;
  }
  return lo;
}

DRGPUM_API drgpum_status drgpum_merge_peers(drgpum_ctx* ctx, void* const* h_peer_ws, uint32_t n_peers,
                                            uint32_t rank, void* stream) {
  if (!ctx) return DRGPUM_EINVAL;
  if (ctx->state < S_BOUND) return fail(ctx, DRGPUM_ESTATE, "merge_peers before workspace_bind");
  if (ctx->consumed) return fail(ctx, DRGPUM_ESTATE, "merge_peers after a consuming finalize: reset first");
  if (drgpum_status _d = set_device(ctx)) return _d;
  MergePeersParams q{};
  if (drgpum_status e = check_peers(ctx, "merge_peers", h_peer_ws, n_peers, rank, q.peer)) return e;
  q.n_peers = n_peers;
  q.rank = rank;
  q.or_off = ctx->L.orw;
  q.first_off = ctx->L.first;
  q.last_off = ctx->L.last;
  q.ctr_off = ctx->L.ctr;
  // the OR-word section is padded to 256 B (zero in every shadow), so the
  // slices can be rounded to whole 16-B vectors
  const uint64_t w4 = (ctx->bitmap_words + ctx->hit_words + 3) / 4 * 4;
  const uint64_t sw = ((w4 + n_peers - 1) / n_peers + 3) / 4 * 4;
  q.w_lo = std::min<uint64_t>(uint64_t(rank) * sw, w4);
  q.w_hi = std::min<uint64_t>(q.w_lo + sw, w4);
  const uint64_t so = (ctx->n_obj + n_peers - 1) / n_peers;
  q.o_lo = std::min<uint64_t>(uint64_t(rank) * so, ctx->n_obj);
  q.o_hi = std::min<uint64_t>(q.o_lo + so, ctx->n_obj);
  ctx->launches += launch_merge_peers(q, ctx->num_sms, as_stream(stream));
  ctx->final_valid = false;
  ctx->owned = ctx->gathered = false;
  CK(cudaGetLastError());
  return DRGPUM_OK;
}

static drgpum_status merge_owned_impl(drgpum_ctx* ctx, void* const* h_peer_ws, uint32_t n_peers,
                                      uint32_t rank, void* d_mc, void* stream);

DRGPUM_API drgpum_status drgpum_merge_peers_owned(drgpum_ctx* ctx, void* const* h_peer_ws,
                                                  uint32_t n_peers, uint32_t rank, void* stream) {
  return merge_owned_impl(ctx, h_peer_ws, n_peers, rank, nullptr, stream);
}

DRGPUM_API drgpum_status drgpum_merge_peers_owned_nvls(drgpum_ctx* ctx, void* const* h_peer_ws,
                                                       uint32_t n_peers, uint32_t rank, void* d_mc_ws,
                                                       void* stream) {
  if (ctx && (!d_mc_ws || reinterpret_cast<uintptr_t>(d_mc_ws) % kAlign))
    return fail(ctx, DRGPUM_EINVAL, "merge_peers_owned_nvls: multicast address NULL or not 256-B aligned");
  return merge_owned_impl(ctx, h_peer_ws, n_peers, rank, d_mc_ws, stream);
}

static drgpum_status merge_owned_impl(drgpum_ctx* ctx, void* const* h_peer_ws, uint32_t n_peers,
                                      uint32_t rank, void* d_mc, void* stream) {
  if (!ctx) return DRGPUM_EINVAL;
  if (ctx->state < S_BOUND) return fail(ctx, DRGPUM_ESTATE, "merge_peers_owned before workspace_bind");
  if (ctx->consumed) return fail(ctx, DRGPUM_ESTATE, "merge_peers_owned after a consuming finalize: reset first");
  if (drgpum_status _d = set_device(ctx)) return _d;
  MergeOwnedParams q{};
  if (drgpum_status e = check_peers(ctx, "merge_peers_owned", h_peer_ws, n_peers, rank, q.peer)) return e;
  q.n_peers = n_peers;
  q.rank = rank;
  q.or_off = ctx->L.orw;
  q.first_off = ctx->L.first;
  q.last_off = ctx->L.last;
  q.ctr_off = ctx->L.ctr;
  const uint64_t lo = owned_cut(ctx, rank, n_peers), hi = owned_cut(ctx, rank + 1, n_peers);
  auto bw = [&](uint64_t o) { return o < ctx->n_obj ? ctx->layout[o].bitmap_word : ctx->bitmap_words; };
  auto hw = [&](uint64_t o) { return ctx->bitmap_words + (o < ctx->n_obj ? ctx->layout[o].hit_word : ctx->hit_words); };
  q.b_lo = bw(lo); q.b_hi = bw(hi);   // multiples of 4 (every bitmap is padded to 4 words)
  q.h_lo = hw(lo); q.h_hi = hw(hi);
  q.o_lo = lo; q.o_hi = hi;
  q.tiles = at<Tile>(ctx, ctx->L.tiles);
  q.t_lo = ctx->tile_off[lo];
  q.t_hi = ctx->tile_off[hi];
  q.objs = at<DevObj>(ctx, ctx->L.objs);
  q.n_hit = at<uint32_t>(ctx, ctx->L.n_hit);
  q.pmask = at<unsigned long long>(ctx, ctx->L.pmask);
  q.mc = static_cast<uint8_t*>(d_mc);
#if DRGPUM_SPARSE_MERGE
  ctx->launches += launch_merge_owned_sparse(q, ctx->num_sms, as_stream(stream));
#else
  ctx->launches += launch_merge_owned(q, ctx->num_sms, as_stream(stream));
#endif
  CK(cudaGetLastError());
  ctx->final_valid = false;
  ctx->owned = true;
  ctx->gathered = false;
  ctx->own_lo = lo; ctx->own_hi = hi; ctx->own_P = n_peers; ctx->own_rank = rank;
  return DRGPUM_OK;
}

DRGPUM_API drgpum_status drgpum_gather_peers(drgpum_ctx* ctx, void* const* h_peer_ws,
                                             uint32_t n_peers, uint32_t rank, void* stream) {
  if (!ctx) return DRGPUM_EINVAL;
  if (ctx->state < S_BOUND) return fail(ctx, DRGPUM_ESTATE, "gather_peers before workspace_bind");
  if (drgpum_status _d = set_device(ctx)) return _d;
  GatherParams q{};
  if (drgpum_status e = check_peers(ctx, "gather_peers", h_peer_ws, n_peers, rank, q.peer)) return e;
  if (!ctx->owned || !ctx->final_valid)
    return fail(ctx, DRGPUM_ESTATE, "gather_peers needs merge_peers_owned then finalize");
  if (n_peers != ctx->own_P || rank != ctx->own_rank)
    return fail(ctx, DRGPUM_EINVAL, "gather_peers: n_peers / rank differ from merge_peers_owned");
  static_assert(sizeof(drgpum_object_stats_t) % 4 == 0 && sizeof(drgpum_pattern_report_t) % 4 == 0,
                "gather copies u32 words");
  q.n_peers = n_peers;
  q.rank = rank;
  q.stats_off = ctx->L.stats;
  q.s_lo = ctx->own_lo * sizeof(drgpum_object_stats_t);
  q.s_hi = ctx->own_hi * sizeof(drgpum_object_stats_t);
  q.reports_off = ctx->L.reports;
  q.r_lo = ctx->own_lo * sizeof(drgpum_pattern_report_t);
  q.r_hi = ctx->own_hi * sizeof(drgpum_pattern_report_t);
  q.ctr_off = ctx->L.ctr;
  q.cons_off = ctx->L.cons;
  ctx->launches += launch_gather_peers(q, ctx->num_sms, as_stream(stream));
  CK(cudaGetLastError());
  ctx->gathered = true;
  return DRGPUM_OK;
}

DRGPUM_API drgpum_status drgpum_finalize(drgpum_ctx* ctx, const drgpum_thresholds_t* th, void* stream) {
  if (!ctx) return DRGPUM_EINVAL;
  if (ctx->state < S_BOUND) return fail(ctx, DRGPUM_ESTATE, "finalize before workspace_bind");
  if (drgpum_status _d = set_device(ctx)) return _d;
  drgpum_thresholds_t t = th ? *th : drgpum_thresholds_t{2, 80, 80};
  cudaStream_t st = as_stream(stream);
  FinalParams p;
  p.orw = at<uint32_t>(ctx, ctx->L.orw);
  p.tiles = at<Tile>(ctx, ctx->L.tiles);
  p.tile_part = at<BitMonoid>(ctx, ctx->L.tile_part);
  p.n_tiles = ctx->tiles.size();
  p.groups = at<Group>(ctx, ctx->L.groups);
  p.group_part = at<BitMonoid>(ctx, ctx->L.group_part);
  p.n_groups = ctx->groups.size();
  p.group_off = at<uint32_t>(ctx, ctx->L.group_off);
  p.objs = at<DevObj>(ctx, ctx->L.objs);
  p.first = at<uint32_t>(ctx, ctx->L.first);
  p.last = at<uint32_t>(ctx, ctx->L.last);
  p.acc_ts = at<uint32_t>(ctx, ctx->L.acc_ts);
  p.acc_cs = at<uint8_t>(ctx, ctx->L.acc_cs);
  p.n_hit = at<uint32_t>(ctx, ctx->L.n_hit);
  p.n_acc = ctx->n_acc;
  p.n_obj = ctx->n_obj;
  p.ti_min_idle = t.ti_min_idle;
  p.oa_pct = t.oa_accessed_pct;
  p.frag_pct = t.oa_frag_pct;
  p.stats = ctx->ws + ctx->L.stats;
  p.reports = ctx->ws + ctx->L.reports;
  p.ctr = at<unsigned long long>(ctx, ctx->L.ctr);
  p.o_lo = ctx->owned ? ctx->own_lo : 0;
  p.o_hi = ctx->owned ? ctx->own_hi : ctx->n_obj;
  p.t_lo = ctx->tile_off[p.o_lo];
  p.t_hi = ctx->tile_off[p.o_hi];
  p.g_lo = ctx->group_off[p.o_lo];
  p.g_hi = ctx->group_off[p.o_hi];
  if (ctx->small_prefix.size() != ctx->n_obj + 1) {   // objects object_finalize folds lane by lane
    ctx->small_prefix.assign(ctx->n_obj + 1, 0);
    for (uint64_t o = 0; o < ctx->n_obj; ++o)
      ctx->small_prefix[o + 1] = ctx->small_prefix[o] +
          (ctx->group_off[o + 1] - ctx->group_off[o] <= 1 && (2ull * ctx->n_hit[o] + 31) / 32 <= kLaneHitWords);
  }
  p.n_small = ctx->small_prefix[p.o_hi] - ctx->small_prefix[p.o_lo];
  // consumed bitmaps: the tile / group monoids of the consuming finalize are
  // still in place, only the classification runs again
  p.skip_tiles = ctx->consumed;
  p.consume = ctx->fin_consume && !ctx->owned && !ctx->consumed;
  ctx->launches += launch_finalize(p, ctx->num_sms, st);
  if (p.consume) ctx->consumed = true;
  ctx->gathered = false;
  CK(cudaGetLastError());
  ctx->final_valid = true;
  ctx->final_th = t;
  return DRGPUM_OK;
}

static bool same_th(const drgpum_thresholds_t& a, const drgpum_thresholds_t& b) {
  return a.ti_min_idle == b.ti_min_idle && a.oa_accessed_pct == b.oa_accessed_pct &&
         a.oa_frag_pct == b.oa_frag_pct;
}

DRGPUM_API drgpum_status drgpum_object_stats(drgpum_ctx* ctx, drgpum_object_stats_t* h_out,
                                             drgpum_counters_t* h_ctr, void* stream) {
  if (!ctx) return DRGPUM_EINVAL;
  if (ctx->state < S_BOUND) return fail(ctx, DRGPUM_ESTATE, "object_stats before workspace_bind");
  if (drgpum_status _d = set_device(ctx)) return _d;
  cudaStream_t st = as_stream(stream);
  if (ctx->owned && !(ctx->final_valid && ctx->gathered))
    return fail(ctx, DRGPUM_ESTATE, "object_stats after merge_peers_owned needs finalize + gather_peers");
  if (!ctx->final_valid) {
    drgpum_status s = drgpum_finalize(ctx, &ctx->final_th, stream);
    if (s != DRGPUM_OK) return s;
  }
  if (h_out && ctx->n_obj)
    CK(cudaMemcpyAsync(h_out, ctx->ws + ctx->L.stats, sizeof(drgpum_object_stats_t) * ctx->n_obj,
                       cudaMemcpyDeviceToHost, st));
  unsigned long long c[C_SLOTS];
  CK(cudaMemcpyAsync(c, ctx->ws + ctx->L.ctr, sizeof c, cudaMemcpyDeviceToHost, st));
  CK(cudaStreamSynchronize(st));
  if (h_ctr) {
    h_ctr->records = c[C_RECORDS];
    h_ctr->attributed = c[C_ATTRIBUTED];
    h_ctr->unattributed = c[C_UNATTRIBUTED];
    h_ctr->clipped = c[C_CLIPPED];
    h_ctr->invalid = c[C_INVALID];
  }
  return DRGPUM_OK;
}

DRGPUM_API drgpum_status drgpum_patterns(drgpum_ctx* ctx, const drgpum_thresholds_t* th,
                                         drgpum_pattern_report_t* h_out, void* stream) {
  if (!ctx) return DRGPUM_EINVAL;
  if (ctx->state < S_BOUND) return fail(ctx, DRGPUM_ESTATE, "patterns before workspace_bind");
  if (drgpum_status _d = set_device(ctx)) return _d;
  drgpum_thresholds_t t = th ? *th : drgpum_thresholds_t{2, 80, 80};
  cudaStream_t st = as_stream(stream);
  if (ctx->owned && !(ctx->final_valid && ctx->gathered && same_th(t, ctx->final_th)))
    return fail(ctx, DRGPUM_ESTATE, "patterns after merge_peers_owned needs finalize (same thresholds) + gather_peers");
  if (!ctx->final_valid || !same_th(t, ctx->final_th)) {
    drgpum_status s = drgpum_finalize(ctx, &t, stream);
    if (s != DRGPUM_OK) return s;
  }
  if (h_out && ctx->n_obj)
    CK(cudaMemcpyAsync(h_out, ctx->ws + ctx->L.reports, sizeof(drgpum_pattern_report_t) * ctx->n_obj,
                       cudaMemcpyDeviceToHost, st));
  CK(cudaStreamSynchronize(st));
  return DRGPUM_OK;
}

DRGPUM_API drgpum_status drgpum_consistency_errors(drgpum_ctx* ctx, uint64_t* h_errors, void* stream) {
  if (!ctx || !h_errors) return DRGPUM_EINVAL;
  if (ctx->state < S_BOUND) return DRGPUM_ESTATE;
  if (drgpum_status _d = set_device(ctx)) return _d;
  cudaStream_t st = as_stream(stream);
  unsigned long long c[C_SLOTS], per_rank[kMaxPeers];
  CK(cudaMemcpyAsync(c, ctx->ws + ctx->L.ctr, sizeof c, cudaMemcpyDeviceToHost, st));
  CK(cudaMemcpyAsync(per_rank, ctx->ws + ctx->L.cons, sizeof per_rank, cudaMemcpyDeviceToHost, st));
  CK(cudaStreamSynchronize(st));
  if (ctx->owned && ctx->gathered) {   // every rank's count of its own objects
    uint64_t sum = 0;
    for (uint32_t r = 0; r < ctx->own_P; ++r) sum += per_rank[r];
    *h_errors = sum;
  } else {
    *h_errors = c[C_CONSISTENCY];
  }
  return DRGPUM_OK;
}

DRGPUM_API drgpum_status drgpum_path_stats(drgpum_ctx* ctx, uint64_t out[4], void* stream) {
  if (!ctx || !out) return DRGPUM_EINVAL;
  if (ctx->state < S_BOUND) return DRGPUM_ESTATE;
  if (drgpum_status _d = set_device(ctx)) return _d;
  cudaStream_t st = as_stream(stream);
  unsigned long long c[C_SLOTS];
  CK(cudaMemcpyAsync(c, ctx->ws + ctx->L.ctr, sizeof c, cudaMemcpyDeviceToHost, st));
  CK(cudaStreamSynchronize(st));
  out[0] = c[C_TILES_AFFINE_UNION];
  out[1] = c[C_TILES_AFFINE_WORDS];
  out[2] = c[C_TILES_FAST];
  out[3] = c[C_TILES_SLOW];
  return DRGPUM_OK;
}

DRGPUM_API drgpum_status drgpum_redundant_alloc(drgpum_ctx* ctx, uint32_t pct, uint32_t* reuser,
                                                uint32_t* donor, uint64_t cap, uint64_t* n_pairs,
                                                void* stream) {
  if (!ctx || !n_pairs || (cap && (!reuser || !donor))) return DRGPUM_EINVAL;
  if (ctx->state < S_BOUND) return fail(ctx, DRGPUM_ESTATE, "redundant_alloc before workspace_bind");
  if (drgpum_status _d = set_device(ctx)) return _d;
  std::vector<drgpum_object_stats_t> st(ctx->n_obj);
  drgpum_status s = drgpum_object_stats(ctx, st.data(), nullptr, stream);
  if (s != DRGPUM_OK) return s;
  std::vector<uint64_t> sizes(ctx->n_obj);
  std::vector<uint32_t> first(ctx->n_obj), last(ctx->n_obj);
  std::vector<uint8_t> used(ctx->n_obj);
  for (uint64_t o = 0; o < ctx->n_obj; ++o) {
    sizes[o] = ctx->objs[o].size;
    first[o] = st[o].t_first;
    last[o] = st[o].t_last;
    used[o] = st[o].n_access_apis > 0;
  }
  s = drgpum_redundant_pairs(sizes.data(), first.data(), last.data(), used.data(), ctx->n_obj, pct,
                             reuser, donor, cap, n_pairs);
  if (s != DRGPUM_OK) return fail(ctx, s, "redundant_pairs: invalid arguments");
  return DRGPUM_OK;
}

}  // extern "C"

namespace {
// Every object's accessing APIs in invocation order with their read/write
// bits, from the hit rows on the device (CSR: off[n_obj + 1]).
drgpum_status gather_accesses(drgpum_ctx* ctx, cudaStream_t st, std::vector<uint64_t>& off,
                              std::vector<uint32_t>& api, std::vector<uint8_t>& rw) {
  std::vector<uint32_t> hit(ctx->hit_words);
  if (ctx->hit_words)
    CK(cudaMemcpyAsync(hit.data(), ctx->ws + ctx->L.orw + 4 * ctx->bitmap_words, 4 * ctx->hit_words,
                       cudaMemcpyDeviceToHost, st));
  CK(cudaStreamSynchronize(st));
  off.assign(ctx->n_obj + 1, 0);
  api.clear();
  rw.clear();
  for (uint64_t o = 0; o < ctx->n_obj; ++o) {
    const auto& l = ctx->layout[o];
    const uint32_t* row = hit.data() + l.hit_word;
    const uint64_t nw = (2ull * l.n_hit_apis + 31) / 32;
    for (uint64_t w = 0; w < nw; ++w)
      for (uint32_t b = row[w]; b;) {
        const uint32_t slot = uint32_t(w * 16 + (__builtin_ctz(b) >> 1));
        const uint32_t pair = (row[w] >> (2 * (slot & 15))) & 3u;
        b &= ~(3u << (2 * (slot & 15)));
        api.push_back(ctx->acc_ts[l.r_lo + slot]);
        rw.push_back(uint8_t(pair));
      }
    off[o + 1] = api.size();
  }
  return DRGPUM_OK;
}
}  // namespace

extern "C" {

DRGPUM_API drgpum_status drgpum_dependency_graph(drgpum_ctx* ctx, const uint32_t* h_stream,
                                                 uint32_t* h_T, uint32_t* h_src, uint32_t* h_dst,
                                                 uint8_t* h_label, uint64_t cap, uint64_t* n_edges,
                                                 void* stream) {
  if (!ctx || !n_edges || (ctx->n_api && !h_stream) || (cap && !h_src && !h_dst && !h_label))
    return DRGPUM_EINVAL;
  if (ctx->state < S_BOUND) return fail(ctx, DRGPUM_ESTATE, "dependency_graph before workspace_bind");
  if (drgpum_status _d = set_device(ctx)) return _d;
  if (ctx->owned)   // hit rows are merged for this rank's objects only
    return fail(ctx, DRGPUM_ESTATE, "dependency_graph after merge_peers_owned: the hit rows of the other ranks' "
                "objects are not merged here (use merge_peers or merge_or)");
  std::vector<uint64_t> off;
  std::vector<uint32_t> api;
  std::vector<uint8_t> rw;
  drgpum_status s = gather_accesses(ctx, as_stream(stream), off, api, rw);
  if (s != DRGPUM_OK) return s;
  std::vector<drgpum_ms::Edge> e;
  e.reserve(ctx->n_api + 3 * api.size());
  drgpum_ms::stream_edges(h_stream, ctx->n_api, e);
  for (uint64_t o = 0; o < ctx->n_obj; ++o)
    drgpum_ms::object_edges(ctx->objs[o].t_alloc, ctx->objs[o].t_free, api.data() + off[o],
                            rw.data() + off[o], off[o + 1] - off[o], e);
  drgpum_ms::canonicalize(e);
  *n_edges = e.size();
  for (uint64_t k = 0; k < std::min<uint64_t>(cap, e.size()); ++k) {
    if (h_src) h_src[k] = e[k].src;
    if (h_dst) h_dst[k] = e[k].dst;
    if (h_label) h_label[k] = uint8_t(e[k].label);
  }
  if (h_T) {
    if (!drgpum_ms::kahn(ctx->n_api, e, h_T))   // edges only go forward in time
      return fail(ctx, DRGPUM_EINVAL, "dependency graph has a cycle");
  }
  return DRGPUM_OK;
}

DRGPUM_API drgpum_status drgpum_patterns_topo(drgpum_ctx* ctx, const uint32_t* h_T,
                                              const drgpum_thresholds_t* th,
                                              drgpum_pattern_report_t* h_out, void* stream) {
  if (!ctx || !h_out || (ctx->n_api && !h_T)) return DRGPUM_EINVAL;
  if (ctx->state < S_BOUND) return fail(ctx, DRGPUM_ESTATE, "patterns_topo before workspace_bind");
  if (drgpum_status _d = set_device(ctx)) return _d;
  if (ctx->owned)   // hit rows are merged for this rank's objects only
    return fail(ctx, DRGPUM_ESTATE, "patterns_topo after merge_peers_owned: the hit rows of the other ranks' "
                "objects are not merged here (use merge_peers or merge_or)");
  const uint32_t n_api = ctx->n_api;
  for (uint32_t v = 0; v < n_api; ++v)
    if (h_T[v] >= n_api) return fail(ctx, DRGPUM_EINVAL, "T[%u] = %u >= n_api", v, h_T[v]);
  drgpum_thresholds_t t = th ? *th : drgpum_thresholds_t{2, 80, 80};
  drgpum_status s = drgpum_patterns(ctx, &t, h_out, stream);    // time-free flags
  if (s != DRGPUM_OK) return s;
  std::vector<uint64_t> off;
  std::vector<uint32_t> api;
  std::vector<uint8_t> rw;
  s = gather_accesses(ctx, as_stream(stream), off, api, rw);
  if (s != DRGPUM_OK) return s;
  // P[L] = number of APIs with T < L; between(a, b) = P[T_b] - P[T_a + 1]
  std::vector<uint64_t> P(uint64_t(n_api) + 2, 0);
  for (uint32_t v = 0; v < n_api; ++v) ++P[h_T[v] + 1];
  for (uint64_t L = 1; L < P.size(); ++L) P[L] += P[L - 1];
  auto between = [&](uint32_t a, uint32_t b) -> uint64_t {
    const uint32_t ta = h_T[a], tb = h_T[b];
    return tb > ta ? P[tb] - P[ta + 1] : 0;
  };
  constexpr uint32_t kTime = DRGPUM_EA | DRGPUM_LD | DRGPUM_TI | DRGPUM_DW;
  std::vector<uint32_t> idx;
  for (uint64_t o = 0; o < ctx->n_obj; ++o) {
    drgpum_pattern_report_t& r = h_out[o];
    r.flags &= ~kTime;
    r.ea_distance = r.ld_distance = r.ti_ranges = r.ti_max_idle = r.dw_pairs = 0;
    r.ti_total_idle = 0;
    const uint64_t n = off[o + 1] - off[o];
    if (!n) continue;
    idx.resize(n);
    std::iota(idx.begin(), idx.end(), uint32_t(off[o]));
    std::sort(idx.begin(), idx.end(), [&](uint32_t a, uint32_t b) {
      const uint32_t ta = h_T[api[a]], tb = h_T[api[b]];
      return ta != tb ? ta < tb : api[a] < api[b];
    });
    const auto& ob = ctx->objs[o];
    const uint32_t f = api[idx.front()], l = api[idx.back()];
    if (between(ob.t_alloc, f) >= 1) {                                   // Def 3.1
      r.flags |= DRGPUM_EA;
      r.ea_distance = h_T[f] - h_T[ob.t_alloc];
    }
    if (ob.t_free != DRGPUM_NEVER && between(l, ob.t_free) >= 1) {       // Def 3.2
      r.flags |= DRGPUM_LD;
      r.ld_distance = h_T[ob.t_free] - h_T[l];
    }
    for (uint64_t k = 1; k < n; ++k) {
      const uint32_t a = idx[k - 1], b = idx[k];
      const uint64_t g = between(api[a], api[b]);                       // Def 3.6
      if (g >= t.ti_min_idle) {
        ++r.ti_ranges;
        r.ti_max_idle = std::max<uint32_t>(r.ti_max_idle, uint32_t(g));
        r.ti_total_idle += g;
      }
      const uint8_t ka = ctx->kinds[api[a]], kb = ctx->kinds[api[b]];    // Def 3.7
      const bool cs_a = ka == DRGPUM_API_MEMCPY || ka == DRGPUM_API_MEMSET;
      const bool cs_b = kb == DRGPUM_API_MEMCPY || kb == DRGPUM_API_MEMSET;
      if (cs_a && cs_b && (rw[a] & 2) && (rw[b] & 2)) ++r.dw_pairs;
    }
    if (r.ti_ranges) r.flags |= DRGPUM_TI;
    if (r.dw_pairs) r.flags |= DRGPUM_DW;
  }
  return DRGPUM_OK;
}

DRGPUM_API const char* drgpum_last_error(const drgpum_ctx* ctx) {
  if (!ctx) return "null context";
  return ctx->err.c_str();
}

DRGPUM_API void drgpum_destroy(drgpum_ctx* ctx) {
  if (!ctx) return;
  if (ctx->copy_stream) {
    cudaStreamDestroy(ctx->copy_stream);
    for (int i = 0; i < 2; ++i) { cudaEventDestroy(ctx->ev_copied[i]); cudaEventDestroy(ctx->ev_used[i]); }
  }
  delete ctx;
}

DRGPUM_API uint64_t drgpum_launch_count(const drgpum_ctx* ctx) { return ctx ? ctx->launches : 0; }

}  // extern "C"
