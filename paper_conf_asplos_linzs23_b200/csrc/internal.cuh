// Internal types shared by the host library and the sm_100a kernels.
// (Nothing here is shared with oracle/ -- the oracle has its own code.)
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

namespace drgpum {

constexpr uint32_t kNever = 0xFFFFFFFFu;
constexpr uint32_t kNone = 0xFFFFFFFFu;        // "no object" / invalid rank
constexpr int kL1MaxKeys = 512;                // level-1 keys staged in shared memory (4 KB)
constexpr uint32_t kRangeChunkWords = 4096;    // range-expansion work item (16 KB of bitmap)
constexpr uint32_t kTileWords = 1024;          // bitmap reduction tile (4 KB)
constexpr uint32_t kGroupTiles = 32;           // tiles per reduction group
constexpr uint64_t kStageRecords = 1ull << 22; // host-ingest staging chunk (64 MB)

// Object as the attribution kernel sees it: 48 bytes, three 16-B loads.
struct alignas(16) DevObj {
  uint64_t base, end;       // [base, end)
  uint64_t bm_bit;          // global bit index of element 0 (word aligned: multiple of 32)
  uint64_t hit_word;        // global u32 word index of the hit row (inside the OR array)
  uint32_t t_alloc, t_free; // live iff t_alloc < ts < t_free
  uint32_t r_lo;            // access-API rank of the first access API after t_alloc
  uint32_t shift;           // log2(elem_size)
};
static_assert(sizeof(DevObj) == 48, "DevObj layout");

// Segment-index candidate: object id + its t_alloc (candidates of a segment
// are sorted by t_alloc and have disjoint lifetimes).
struct CandEntry { uint32_t obj, t_alloc; };

// Segment entry (16 B): the start address and, when the segment has exactly
// one candidate (the common, reuse-free case), that object and its t_alloc,
// so a lookup resolves in one load per search level.
//   ref = object id (< 2^31), aux = its t_alloc       one candidate
//   ref = kNone                                      no candidate
//   ref = kMultiBit | cand_off, aux = count           several (cand[] by t_alloc)
constexpr uint32_t kMultiBit = 0x80000000u;
struct alignas(16) SegEntry { uint64_t start; uint32_t ref, aux; };
static_assert(sizeof(SegEntry) == 16, "SegEntry layout");

// Chunk-start hint (64 B): the object of the first record of an attribution
// work chunk, resolved for all chunks of a launch at once by
// chunk_hint_kernel (obj = kNone: no live object / invalid record).
struct alignas(16) ChunkHint { DevObj o; uint32_t obj; uint32_t pad[3]; };
static_assert(sizeof(ChunkHint) == 64, "ChunkHint layout");
#ifndef DRGPUM_CHUNK_MAX_SHIFT_SMALL
#define DRGPUM_CHUNK_MAX_SHIFT_SMALL 15
#endif
constexpr uint32_t kChunkMaxShiftSmall = DRGPUM_CHUNK_MAX_SHIFT_SMALL;   // big-chunk bound, small-object traces
constexpr uint32_t kHintCap = 1u << 20;          // chunks per launch that get a hint (64 MB)

// Range-expansion queue entry: inclusive global bit range, <= kRangeChunkWords words.
struct RangeEntry { uint64_t bit_lo, bit_hi; };

// Bitmap reduction tile: a run of <= kTileWords words of ONE object.
struct Tile { uint64_t word_lo; uint32_t n_words; uint32_t obj; uint64_t elem_lo; uint64_t n_bits; };
// Reduction group: <= kGroupTiles consecutive tiles of ONE object.
struct Group { uint32_t tile_lo, n_tiles; };

// Bitmap run monoid over a bit sequence.  Positions are
// relative to the start of the sequence; kNoPos when the sequence has no 1.
constexpr uint64_t kNoPos = ~0ull;
struct BitMonoid {
  uint64_t len, pop, lo, hi, pre, suf, best;
};

// Counter slots (u64) at the start of the counters block.
enum : int { C_RECORDS = 0, C_ATTRIBUTED, C_UNATTRIBUTED, C_CLIPPED, C_INVALID,
             C_RQ_OVERFLOW, C_CONSISTENCY, C_RQ_COUNT,
             // diagnostics: 32-record tiles by attribution path
             C_TILES_AFFINE_UNION, C_TILES_AFFINE_WORDS, C_TILES_FAST, C_TILES_SLOW,
             C_WORK,   // attribution work cursor (chunk tickets handed out)
             C_RQ_COUNT_ALT,   // range-queue count of odd-numbered attribute calls
             C_RESERVED14,
             C_SLOTS = 16 };

struct AttrParams {
  const uint4* recs;
  uint64_t n;
  const DevObj* objs;
  const uint64_t* seg_start;
  const uint32_t* seg_cand_off;
  const SegEntry* seg;       // [n_seg]
  const CandEntry* cand;
  const uint64_t* l1;        // every l1_stride-th segment start
  uint32_t n_seg, n_l1, l1_stride, n_api;
  const uint32_t* acc_rank;  // [n_api], kNone for ALLOC/FREE
  uint32_t* orw;             // OR-mergeable words: bitmaps then hit rows
  uint32_t* first;
  uint32_t* last;
  unsigned long long* ctr;
  uint32_t* rfull;           // [n_obj] 1 once a whole-object range was queued (zeroed by the reset)
  RangeEntry* rq;
  uint32_t rq_cap;
  uint32_t rq_slot;          // counter slot of this call's range-queue count (C_RQ_COUNT / _ALT)
  uint32_t chunk_shift;      // log2 of the attribution's big work chunk (set by launch_attribute)
  uint32_t chunk_max_shift;  // its upper bound (objects_load: larger when small objects dominate)
  // guided-tail boundaries of the launch's chunks (records b1 < b2 < b3, chunk
  // indices k1 < k2 < k3; launch_attribute computes them once per launch)
  uint64_t cb1, cb2, cb3, ck1, ck2, ck3;
  const ChunkHint* hints;    // [hint_cap] chunk-start hints (launch_attribute fills them)
  uint32_t hint_cap;         // chunks with a hint in this launch (0: none)
};

// NEXT-3 structured access pass (optional feature).
struct SaRange { uint64_t g_lo, g_hi; uint32_t obj, tag; uint32_t pad[2]; };   // 32 B
struct SaParams {
  AttrParams a;              // records, object table, index, rank table
  uint32_t* owner;           // [sum n_elem] access-rank+1 of the first API touching the element
  const uint64_t* elem_base; // [n_obj] first global element index of each object
  uint32_t* overlap;         // [n_obj] 1 if two APIs touched one element
  SaRange* q;                // large-range queue
  uint32_t q_cap;
  unsigned long long* q_count;
  const uint8_t* in_group;   // [n_api] 1 = the API takes part in the pass [R23]
};

// NEXT-2 non-uniform access frequency pass (optional feature), sort-based:
// every attributed record becomes the element interval it touches, as two
// event keys (rank << pos_bits) | (4*g0) and (rank << pos_bits) | (4*g1+2),
// or one point key (rank << pos_bits) | (4*g+1) for a single element
// (g = global element index, rank = access-API rank); adjacent disjoint
// intervals of a warp's consecutive records are merged first.  An LSD radix
// sort orders the keys by (API, element); a scan of the +1 / -1 events gives
// every element's count within its API, and each run of equal count c over
// len elements adds (len, c*len, c*c*len) to its (object, API) slot.  The
// API of the call's last records may continue in the next call: its events
// are carried over, sorted, and swept when the next call (or a query)
// completes it.
// Single-element intervals (after merging) as ONE key: positions are
// 4*g + type, type 0 = start, 1 = point, 2 = end (0: 2*g start, 2*g+1 end).
#ifndef DRGPUM_FQ_POINTS
#define DRGPUM_FQ_POINTS 1
#endif
constexpr uint64_t kFreqPosMul = DRGPUM_FQ_POINTS ? 4 : 2;
#ifndef DRGPUM_FQ_TILE
#define DRGPUM_FQ_TILE 4096
#endif
constexpr uint32_t kFreqTileKeys = DRGPUM_FQ_TILE;   // radix-sort tile (256 threads x 16 keys)
constexpr uint32_t kFreqRadixBits = 9;          // digit width of the LSD passes (512 bins)
// control words (u64): [0..8) counts / buffer / split, [8..16) per-pass skip
// flags, [16..24) per-pass tile tickets, [32..) per-pass digit totals
constexpr uint32_t kFreqCtlTot = 32;
constexpr uint32_t kFreqMaxDigits = 8;
constexpr uint32_t kFreqCtlWords = kFreqCtlTot + kFreqMaxDigits * (1u << kFreqRadixBits);
constexpr uint32_t kFreqScanItems = 2048;       // entries per block of the digit-offset scan
struct FreqParams {
  AttrParams a;                  // records of this (sub-)call, object table, index, rank table
  const uint64_t* elem_base;     // [n_obj] first global element of each object
  const uint64_t* slot_base;     // [n_obj] first (object, access API) slot of each object
  unsigned long long* acc;       // [n_slots][3] completed APIs: n, S1 = sum f, S2 = sum f^2
  unsigned long long* acc_q;     // [n_slots][3] acc + the carried API (written by queries)
  uint32_t* state;               // [0] bit0 records out of order, bit1 event capacity exceeded;
                                 // [1] last timestamp of the previous call + 1 (0 = none)
  unsigned long long* ctl;       // [0] keys in the current buffer, [1] current buffer, [2] split,
                                 // [8..16) skip flag per radix pass, [16..24) tile tickets,
                                 // [32..) digit totals
  uint64_t* keys0;               // event keys, ping-pong buffers of cap keys
  uint64_t* keys1;
  uint64_t cap;
  uint32_t* hist;                // [bins * max_tiles] per-tile digit counts
  uint32_t* offs;                // [bins * max_tiles] exclusive digit offsets (scanned)
  uint32_t* part;                // [scan blocks] block sums of offs, then of the sweep
  uint64_t max_tiles;
  uint64_t n_obj;
  uint32_t pos_bits, n_digits;
};
struct FreqReduceParams {
  const unsigned long long* acc;
  const uint64_t* slot_base;
  const uint32_t* n_hit;         // [n_obj] slots per object
  const DevObj* objs;
  const uint32_t* acc_ts;
  uint64_t n_obj;
  uint32_t pct;
  uint32_t* out_count;           // [n_obj] APIs at which the object matches NUAF
  uint32_t* out_first;           // [n_obj] first such timestamp (kNever if none)
};

struct FinalParams {
  const uint32_t* orw;
  const Tile* tiles;
  BitMonoid* tile_part;
  uint64_t n_tiles;
  const Group* groups;
  BitMonoid* group_part;
  uint64_t n_groups;
  const uint32_t* group_off;  // [n_obj+1]
  const DevObj* objs;
  const uint32_t* first;
  const uint32_t* last;
  const uint32_t* acc_ts;    // [n_acc]
  const uint8_t* acc_cs;     // [n_acc] 1 if MEMCPY/MEMSET
  const uint32_t* n_hit;     // [n_obj] number of access APIs in the hit row
  uint32_t n_acc;
  uint64_t n_obj;
  uint32_t ti_min_idle, oa_pct, frag_pct;
  void* stats;               // drgpum_object_stats[n_obj]
  void* reports;             // drgpum_pattern_report[n_obj]
  unsigned long long* ctr;
  // the objects this call finalizes ([0, n_obj) unless an owned merge
  // narrowed it) and their tiles / groups
  uint64_t o_lo, o_hi, t_lo, t_hi, g_lo, g_hi;
  uint64_t n_small;          // objects in [o_lo, o_hi) with one bitmap group and <= kLaneHitWords hit words
  bool consume;              // tile_reduce zeroes the bitmap words it reads (reduce-and-clear)
  bool skip_tiles;           // bitmaps consumed earlier: tile / group monoids are already in place
};
constexpr uint32_t kLaneHitWords = 128;   // hit rows a single lane folds in object_finalize (<= 2048 APIs)

// Peer-memory merge (B7'): workspace base pointers of every rank, indexed by rank.
constexpr uint32_t kMaxPeers = 64;
struct MergePeersParams {
  uint8_t* peer[kMaxPeers];
  uint32_t n_peers, rank;
  uint64_t or_off, first_off, last_off, ctr_off;   // byte offsets inside a workspace
  uint64_t w_lo, w_hi;                             // owned OR-word slice (multiples of 4)
  uint64_t o_lo, o_hi;                             // owned object slice
};

// Owned merge (B7''): rank r combines only the shadow of ITS objects
// [o_lo, o_hi) -- bitmap words [b_lo, b_hi) (16-B vectors [b_lo/4, b_hi/4)),
// hit-row words [h_lo, h_hi) of the OR section, first/last -- from every
// peer into its own workspace; rank 0 sums the counters into every peer.
struct MergeOwnedParams {
  uint8_t* peer[kMaxPeers];
  uint32_t n_peers, rank;
  uint64_t or_off, first_off, last_off, ctr_off;
  uint64_t b_lo, b_hi, h_lo, h_hi, o_lo, o_hi;
  // sparse form: the owned objects' tiles [t_lo, t_hi) and per-object masks
  // of the peers whose first[] is set (only those hold nonzero words)
  const Tile* tiles;
  uint64_t t_lo, t_hi;
  const DevObj* objs;
  const uint32_t* n_hit;
  unsigned long long* pmask;   // [n_obj] (this workspace)
  uint8_t* mc;                 // NVLS multicast mapping of the workspaces (nullptr: peer loads only)
};

// Gather (B7''): rank r stores bytes [lo, hi) of the stats and of the
// reports sections (its objects) into every peer, and its consistency count
// into slot r of every peer's per-rank consistency array (a plain store, so
// a re-finalize + re-gather replaces the count instead of adding it again).
struct GatherParams {
  uint8_t* peer[kMaxPeers];
  uint32_t n_peers, rank;
  uint64_t stats_off, s_lo, s_hi, reports_off, r_lo, r_hi, ctr_off, cons_off;
};

// Launchers (return the number of kernels enqueued).
// Set the kernels' attributes on the CURRENT device and return their
// resident blocks per SM (called by workspace_bind; cached in the context).
int attribute_occupancy();
int launch_attribute(const AttrParams& p, int num_sms, int occ, cudaStream_t s);   // p.rq_slot alternates per call
int launch_structured(const SaParams& p, int num_sms, cudaStream_t s);
int launch_frequency(const FreqParams& p, int num_sms, cudaStream_t s);
// queries: acc_q = acc + the carried API's contributions
int launch_frequency_query(const FreqParams& p, uint64_t n_slots, int num_sms, cudaStream_t s);
int launch_frequency_reduce(const FreqReduceParams& p, int num_sms, cudaStream_t s);
int launch_finalize(const FinalParams& p, int num_sms, cudaStream_t s);
int launch_fill_u32(uint32_t* p, uint32_t v, uint64_t n, cudaStream_t s);
int launch_reset(void* ws, uint64_t bytes, uint64_t first_off, uint64_t first_bytes, int num_sms, cudaStream_t s);
// Sparse reset of the OR words: zero the bitmap tiles and hit rows of the
// objects whose first[] is not NEVER (every attributed or merged bit of an
// object comes with a first-use fold, so the others are still all zero).
int launch_reset_touched(uint32_t* orw, const Tile* tiles, uint64_t n_tiles, const DevObj* objs,
                         const uint32_t* n_hit, const uint32_t* first, uint64_t n_obj, bool lane_tiles,
                         int num_sms, cudaStream_t s);
int launch_merge_peers(const MergePeersParams& q, int num_sms, cudaStream_t s);
int launch_merge_owned(const MergeOwnedParams& q, int num_sms, cudaStream_t s);
int launch_merge_owned_sparse(const MergeOwnedParams& q, int num_sms, cudaStream_t s);
int launch_gather_peers(const GatherParams& q, int num_sms, cudaStream_t s);
int launch_merge_or(uint32_t* dst, const uint32_t* src, uint32_t n_src,
                    uint64_t src_stride, uint64_t n_words, int num_sms, cudaStream_t s);

}  // namespace drgpum
