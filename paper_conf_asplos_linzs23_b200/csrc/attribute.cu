// B1 attribute_kernel + B2 range_expand_kernel (sm_100a).
//
// Per record (§5.1 l.238-240, §5.2 l.264-268):
//   A1  stream the 16-B records: each block owns one contiguous record range
//       and a producer lane streams it through a 4-stage shared-memory ring
//       with cp.async.bulk (TMA bulk copy, L2 evict-first), mbarrier-paced;
//       reject invalid records (size 0, ts >= n_api, ts of an ALLOC/FREE API
//       -- footnote 2 l.178 --, addr+size overflow);
//   A2  find the object live at ts that contains addr: each lane caches the
//       last (object, API) it validated; bursts are warp-coalesced, so almost
//       every 32-record tile takes the uniform FAST path (all lanes inside
//       their cached object and API: no search, no liveness/hit work).
//       Otherwise the SLOW path runs the full per-lane algorithm: two-level
//       search of the static segment index (level-1 keys in shared memory,
//       leaves in L2), candidate search by t_alloc (address reuse, R5);
//   A3  clip to the object (R3), element bits (partial elements count, R2),
//       OR into the object's bitmap.  Fast path: when the 32 lanes' bit
//       ranges chain into one contiguous range (sequential sweeps of any
//       access size) the warp writes that union directly, one RED.OR per
//       word; otherwise runs of equal words are merged by a shuffle
//       segmented scan (or not at all when every lane has its own word).
//       Records spanning > 2 words go to the range queue (A3b);
//   A4  fold ts into first (RED.MIN) / last (RED.MAX) and OR the (access API,
//       read|write) bit into the object's hit row -- once per lane per
//       (object, API, rw), in the slow path;
//   A5  count records / attributed / unattributed / clipped / invalid.
#include "internal.cuh"

namespace drgpum {

#define FULL_MASK 0xFFFFFFFFu

// Geometry (macros only for A/B builds, tools/build_variant.sh).  Measured on
// C2 (tools/ab.sh, one box): 8 warps x 3 stages x 4 tiles at 3 blocks/SM
// 0.404 ms; 256-record stages (8 tiles; 2 stages, 4 or 8 warps) 0.414-0.417;
// 4 stages with 6-8 warps 0.405-0.411; 5 stages x 5 warps 0.417.
#ifndef DRGPUM_WARPS
#define DRGPUM_WARPS 8
#endif
#ifndef DRGPUM_STAGES
#define DRGPUM_STAGES 3
#endif
#ifndef DRGPUM_TILES
#define DRGPUM_TILES 4
#endif
#ifndef DRGPUM_MINBLOCKS
#define DRGPUM_MINBLOCKS 3
#endif
constexpr int kConsumerWarps = DRGPUM_WARPS;
constexpr int kAttrThreads = kConsumerWarps * 32;
constexpr int kStages = DRGPUM_STAGES;                       // per-warp ring depth
constexpr int kTilesPerWarp = DRGPUM_TILES;                  // 32-record tiles per stage
constexpr int kWarpRecords = kTilesPerWarp * 32;             // 128 records = 2 KB per stage
// Work units: chunk k of a launch covers records [chunk_start(k),
// chunk_start(k+1)).  Big chunks (fewer cache warm-ups at chunk starts) cover
// the first kBigPct% of the records, small ones the rest (balance).  With
// kStatic, the big part is instead one contiguous range per warp, handed out
// without an atomic (ticket k < W is warp k's range).  Measured on C2 (A/B on
// one box, tools/ab.sh): 8192/4096 at 80% beats 8192/1024 by 6%, uniform 4096
// by 5%, uniform 2048 by 16% (each chunk start costs a cache warm-up through
// the slow path) and the static split by 14% (warps spread over the whole
// trace touch the whole shadow at once: the REDs' L2 working set grows).
#ifndef DRGPUM_CHUNK_BIG
#define DRGPUM_CHUNK_BIG 8192
#endif
#ifndef DRGPUM_CHUNK_SMALL
#define DRGPUM_CHUNK_SMALL 4096
#endif
#ifndef DRGPUM_BIG_PCT
#define DRGPUM_BIG_PCT 85
#endif
#ifndef DRGPUM_STATIC
#define DRGPUM_STATIC 0
#endif
#ifndef DRGPUM_FETCH_V2
#define DRGPUM_FETCH_V2 1   // per-stage fetch bookkeeping as records-left + next address (A/B macro)
#endif
#ifndef DRGPUM_TICKET_AHEAD
#define DRGPUM_TICKET_AHEAD 2   // stages before a chunk's end at which the next chunk's ticket is taken
#endif
#ifndef DRGPUM_TAIL
#define DRGPUM_TAIL 1   // guided tail (below): C2 0.389 -> 0.381 ms with kBigPct 85; C3 within noise
#endif
constexpr uint64_t kChunkBig = DRGPUM_CHUNK_BIG, kChunkSmall = DRGPUM_CHUNK_SMALL;
constexpr uint64_t kBigPct = DRGPUM_BIG_PCT;
constexpr bool kStatic = DRGPUM_STATIC != 0;
// Big chunks grow with the records per warp (launch_attribute: 2^chunk_shift
// records, from 8192 while every warp still gets at least kChunksPerWarp of
// them, up to AttrParams::chunk_max_shift: 2^15 when most bitmap tiles are
// small -- the per-warp scratch path, C5 -- else 2^13).  A/B on one box
// (DESIGN.md section 6): 8192 -> 16384 -> 32768 records per chunk take C5
// (302k records per warp and launch) from 47.6 to 44.3 to 42.9 ms and C4
// from 10.54 to 10.29 to 10.21 ms, but C3 from 2.86 to 3.52 to 4.10 ms; C2
// (28k per warp) keeps 8192 either way.  C3's loss is one straggler chunk of slow tiles
// (DESIGN.md section 6), so for any trace a big chunk may also grow while it
// stays within a quarter of the tail every warp gets (DRGPUM_TAIL_GUARD):
// C4 (1.13M records per warp) 10.58 -> 10.25 ms, C3 unchanged.
#ifndef DRGPUM_CHUNK_MAX_SHIFT
#define DRGPUM_CHUNK_MAX_SHIFT 13
#endif
#ifndef DRGPUM_CHUNKS_PER_WARP
#define DRGPUM_CHUNKS_PER_WARP 8
#endif
static_assert((kChunkBig & (kChunkBig - 1)) == 0, "big chunks are powers of two");
#ifndef DRGPUM_TAIL_GUARD
#define DRGPUM_TAIL_GUARD 4   // big chunks <= (tail records per warp) / this, whatever the objects (0: off)
#endif
uint32_t attribute_chunk_shift(uint64_t n, uint64_t n_warps, uint32_t max_shift) {
  uint32_t shift = 0;
  for (uint64_t c = kChunkBig; (c >> 1) != 0; c >>= 1) ++shift;   // log2(kChunkBig)
  const uint32_t cap = max_shift > DRGPUM_CHUNK_MAX_SHIFT ? max_shift : DRGPUM_CHUNK_MAX_SHIFT;
  const uint64_t per = n_warps ? n / n_warps : n;
  while (shift < cap && per >= (2ull << shift) * DRGPUM_CHUNKS_PER_WARP) ++shift;
  // any trace: a big chunk may grow while it stays within a quarter of the
  // small-chunk tail every warp gets ((100 - kBigPct)% of its records), so
  // one chunk of slow tiles (C3's straggler) is absorbed by the tail
  if (DRGPUM_TAIL_GUARD)
    while (shift < kChunkMaxShiftSmall &&
           (2ull << shift) * DRGPUM_TAIL_GUARD <= per / 100 * (100 - kBigPct)) ++shift;
  return shift;
}
// guided tail: big chunks for the first kBigPct%, then 4096 up to 95%, 2048
// up to 98.5%, 1024 to the end (smaller pieces where the last warps finish,
// big ones where chunk-start warm-ups would dominate).  The boundaries are
// computed once per launch on the host (chunk_bounds): a chunk start in the
// kernel is a few compares and one multiply-add (the in-kernel 64-bit
// divisions by 100 / 1000 were a dependent chain on lane 0 at every chunk).
void chunk_bounds(AttrParams& p) {
  const uint64_t n = p.n;
  const uint32_t cs = p.chunk_shift;
  const uint64_t b1 = ((n / 100 * kBigPct) >> cs) << cs;
  const uint64_t e2 = n / 1000 * 950, e3 = n / 1000 * 985;
  const uint64_t b2 = b1 + (e2 - (e2 < b1 ? e2 : b1)) / 4096 * 4096;
  const uint64_t b3 = b2 + (e3 - (e3 < b2 ? e3 : b2)) / 2048 * 2048;
  p.cb1 = b1; p.cb2 = b2; p.cb3 = b3;
  p.ck1 = b1 >> cs; p.ck2 = p.ck1 + (b2 - b1) / 4096; p.ck3 = p.ck2 + (b3 - b2) / 2048;
}
__device__ __forceinline__ uint64_t chunk_start(uint64_t k, const AttrParams& p, uint32_t n_warps) {
  if (kStatic) {
    const uint64_t per = p.n / 100 * kBigPct / n_warps;
    return k <= n_warps ? k * per : n_warps * per + (k - n_warps) * kChunkSmall;
  }
#if DRGPUM_TAIL
  if (k <= p.ck1) return k << p.chunk_shift;
  if (k <= p.ck2) return p.cb1 + (k - p.ck1) * 4096;
  if (k <= p.ck3) return p.cb2 + (k - p.ck2) * 2048;
  return p.cb3 + (k - p.ck3) * 1024;
#else
  return k <= p.ck1 ? k << p.chunk_shift : (p.ck1 << p.chunk_shift) + (k - p.ck1) * kChunkSmall;
#endif
}

// ------------------------------------------------------------------ PTX helpers
// Shared memory is addressed through 32-bit shared-window addresses (no
// generic -> shared conversion in the loop).
__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}
__device__ __forceinline__ void mbar_init(uint32_t bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(bar), "r"(count));
}
__device__ __forceinline__ void mbar_arrive(uint32_t bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(bar) : "memory");
}
__device__ __forceinline__ void mbar_arrive_expect_tx(uint32_t bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(bytes) : "memory");
}
// bar + OFF: the constant offset stays an immediate of the instruction (no
// hoisted, register-resident base per field)
#ifndef DRGPUM_MBAR_TEST
#define DRGPUM_MBAR_TEST 0   // A/B: spin on the non-blocking test_wait instead of try_wait
#endif
template <uint32_t OFF>
__device__ __forceinline__ void mbar_wait(uint32_t bar, uint32_t parity) {
  uint32_t done;
  do {
#if DRGPUM_MBAR_TEST
    asm volatile(
        "{ .reg .pred p; mbarrier.test_wait.parity.shared::cta.b64 p, [%1+%3], %2; selp.u32 %0, 1, 0, p; }"
        : "=r"(done) : "r"(bar), "r"(parity), "n"(OFF) : "memory");
#else
    asm volatile(
        "{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1+%3], %2; selp.u32 %0, 1, 0, p; }"
        : "=r"(done) : "r"(bar), "r"(parity), "n"(OFF) : "memory");
#endif
  } while (!done);
}
__device__ __forceinline__ void tma_load_1d(uint32_t dst, const void* gsrc, uint32_t bytes, uint32_t bar,
                                            uint64_t policy) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1], %2, [%3], %4;"
      ::"r"(dst), "l"(gsrc), "r"(bytes), "r"(bar), "l"(policy) : "memory");
}
__device__ __forceinline__ uint64_t evict_first_policy() {
  uint64_t p;
  asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
  return p;
}
__device__ __forceinline__ uint4 lds128(uint32_t saddr) {
  uint4 r;
  asm volatile("ld.shared.v4.u32 {%0,%1,%2,%3}, [%4];"
               : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "r"(saddr));
  return r;
}
template <uint32_t OFF>
__device__ __forceinline__ uint32_t lds32(uint32_t a) {
  uint32_t v;
  asm volatile("ld.shared.u32 %0, [%1+%2];" : "=r"(v) : "r"(a), "n"(OFF) : "memory");
  return v;
}
__device__ __forceinline__ void sts32(uint32_t a, uint32_t v) {
  asm volatile("st.shared.u32 [%0], %1;" ::"r"(a), "r"(v) : "memory");
}
__device__ __forceinline__ uint64_t lds64(uint32_t a) {
  uint64_t v;
  asm volatile("ld.shared.u64 %0, [%1];" : "=l"(v) : "r"(a) : "memory");
  return v;
}
__device__ __forceinline__ void sts64(uint32_t a, uint64_t v) {
  asm volatile("st.shared.u64 [%0], %1;" ::"r"(a), "l"(v) : "memory");
}
template <uint32_t OFF>
__device__ __forceinline__ void red_shared_add(uint32_t a, uint32_t v) {
  asm volatile("red.shared.add.u32 [%0+%2], %1;" ::"r"(a), "r"(v), "n"(OFF) : "memory");
}
// Work cursor: u32 chunk tickets (the low half of the u64 counter slot).  The
// returned ticket is consumed one chunk later, so the atomic's latency hides
// behind a chunk of work.  Called by lane 0 only; the address is offset by
// %laneid * 8 (= 0 there) so that ptxas cannot prove it warp-uniform and does
// not turn the atomic into a warp-aggregated one whose broadcast would wait
// for the result right away.
__device__ __forceinline__ uint32_t take_ticket(unsigned long long* slot) {
  uint32_t k;
  asm volatile(
      "{ .reg .u32 l; .reg .u64 o, a; mov.u32 l, %%laneid; mul.wide.u32 o, l, 8; add.u64 a, %1, o;"
      " atom.relaxed.gpu.global.add.u32 %0, [a], 1; }"
      : "=r"(k) : "l"(slot) : "memory");
  return k;
}

__device__ __forceinline__ uint32_t bits_mask(uint32_t b0, uint32_t b1) {  // bits b0..b1 inclusive
  return (0xFFFFFFFFu >> (31 - b1)) & (0xFFFFFFFFu << b0);
}

// Fire-and-forget global reductions (SASS REDG): OR/MIN/MAX are idempotent and
// commutative, results are only read after the kernel, so relaxed gpu scope.
#ifdef DRGPUM_DIAG_NORED
// Diagnostic build only (tools/build_variant.sh NAME -DDRGPUM_DIAG_NORED=1):
// every OR-RED is issued under a predicate that is false at run time, so the
// instruction stream is unchanged and only the RED traffic through L1TEX/L2
// disappears.  C2: 0.404 -> 0.303 ms -- the price of ~28M scattered RED
// sectors (profiles/r01_c2_r40.md).  Results are wrong by construction.
__constant__ uint32_t c_red_on = 0;
__device__ __forceinline__ void red_or(uint32_t* a, uint32_t v) {
  asm volatile("{ .reg .pred q; setp.ne.u32 q, %2, 0; @q red.relaxed.gpu.global.or.b32 [%0], %1; }"
               ::"l"(a), "r"(v), "r"(c_red_on) : "memory");
}
#else
__device__ __forceinline__ void red_or(uint32_t* a, uint32_t v) {
  asm volatile("red.relaxed.gpu.global.or.b32 [%0], %1;" ::"l"(a), "r"(v) : "memory");
}
#endif
__device__ __forceinline__ void red_min(uint32_t* a, uint32_t v) {
  asm volatile("red.relaxed.gpu.global.min.u32 [%0], %1;" ::"l"(a), "r"(v) : "memory");
}
__device__ __forceinline__ void red_max(uint32_t* a, uint32_t v) {
  asm volatile("red.relaxed.gpu.global.max.u32 [%0], %1;" ::"l"(a), "r"(v) : "memory");
}

// ------------------------------------------------------------------ warp helpers
// Warp segmented inclusive scan over runs of adjacent lanes with equal keys.
// Returns the run-reduced value in the run's last lane (tail = true there).
template <typename Op>
__device__ __forceinline__ uint32_t seg_scan(uint64_t key, uint32_t v, int lane, bool& tail, Op op) {
  const uint64_t pk = __shfl_up_sync(FULL_MASK, key, 1);
  const bool head = lane == 0 || pk != key;
  const uint32_t heads = __ballot_sync(FULL_MASK, head);
  const int start = 31 - __clz(heads & (FULL_MASK >> (31 - lane)));
#pragma unroll
  for (int d = 1; d < 32; d <<= 1) {
    const uint32_t t = __shfl_up_sync(FULL_MASK, v, d);
    if (lane - d >= start) v = op(v, t);
  }
  tail = lane == 31 || ((heads >> (lane + 1)) & 1u);
  return v;
}

struct OpOr { __device__ uint32_t operator()(uint32_t a, uint32_t b) const { return a | b; } };
struct OpMin { __device__ uint32_t operator()(uint32_t a, uint32_t b) const { return a < b ? a : b; } };
struct OpMax { __device__ uint32_t operator()(uint32_t a, uint32_t b) const { return a > b ? a : b; } };

constexpr uint64_t kNoKey = ~0ull;

// OR masks into words: one RED per run of adjacent lanes sharing a word when
// runs are long, one RED per lane when (almost) every lane has its own word.
__device__ __forceinline__ void warp_or_words(uint32_t* words, uint64_t key, uint32_t m, int lane) {
  const uint64_t pk = __shfl_up_sync(FULL_MASK, key, 1);
  const uint32_t heads = __ballot_sync(FULL_MASK, lane == 0 || pk != key);
  if (heads == 1u) {  // one word for the whole warp
    const uint32_t v = __reduce_or_sync(FULL_MASK, m);
    if (lane == 0 && key != kNoKey && v) red_or(words + key, v);
    return;
  }
  if (__popc(heads) > 16) {  // mostly distinct words: OR is idempotent, just RED
    if (key != kNoKey && m) red_or(words + key, m);
    return;
  }
  bool tail;
  const uint32_t v = seg_scan(key, m, lane, tail, OpOr());
  if (tail && key != kNoKey && v) red_or(words + key, v);
}

// ------------------------------------------------------------------ lane state
// Per-lane object cache.  The authoritative copy lives in SHARED memory (one
// per thread) and only the out-of-line slow paths touch it; the fast paths run
// on a register mirror of the five fields they need, so the slow-path state
// costs no registers (this is what lets three blocks share an SM).
struct SlowCache {                       // 56 B
  uint64_t base, size;                   // cached object: [base, base+size)
  uint64_t bm_word, hit_word;            // its first bitmap word; its hit-row word
  uint32_t t_alloc, t_free, r_lo, shift, obj;
  uint32_t meta;                         // ts|w<<31 whose first/last/hit work is done
};
struct FastCache { uint64_t base, size, bm_word; uint32_t shift, meta; bool sc; };   // sc: scratch_ok

// per warp, shared memory: record counters of the slow paths and the tile
// counts by path (diagnostics; shared-memory REDs keep them out of registers)
struct WarpCounts { uint32_t rec, attr, unattr, clip, inval, ovf, aff_u, aff_w, fast, slow; };

// Per-warp shared region, addressed through ONE 32-bit shared address: the
// ring stages, their barriers and record counts, lane 0's fetch position and
// the counters.
// Small objects (bitmap <= kScratchWords words, i.e. <= 4096 elements): the
// fast tiers OR their per-record masks into a per-warp shared-memory copy of
// the object's bitmap (RED.shared) instead of global REDs; the copy is
// flushed -- one global RED per nonzero word, coalesced -- when the warp's
// object changes and at the end of the kernel.  A burst of thousands of
// scattered records over a small object then costs a handful of global RED
// sectors instead of one per record.  Exact: OR is idempotent and
// commutative, every scratch bit reaches global memory before the kernel ends.
#ifndef DRGPUM_SCRATCH
#define DRGPUM_SCRATCH 128
#endif
constexpr uint32_t kScratchWords = DRGPUM_SCRATCH;
// Large objects: the same scratch as a 128-word WINDOW of the object (base
// aligned to 64 words) for per-record tiers whose records span < 64 words --
// strided sweeps with small strides; consecutive stages of a sweep share the
// window, flushed when it moves.  C2 0.404 -> 0.392 ms (A/B, tools/ab.sh).
#ifndef DRGPUM_WINDOW
#define DRGPUM_WINDOW 1
#endif
// Small objects' contiguous unions (affine tier) and chained tiles also go
// through the scratch (A/B macro).
#ifndef DRGPUM_UNION_SCRATCH
#define DRGPUM_UNION_SCRATCH 1
#endif
constexpr uint64_t kNoScratch = ~0ull;

struct alignas(16) WarpSmem {
  uint4 ring[kStages][kWarpRecords];   // 3 x 2 KB stages
  uint4 hint[kStages][4];              // chunk-start hint of the stage (ChunkHint), when flagged
  uint32_t scratch[kScratchWords > 0 ? kScratchWords : 4];   // small-object bitmap copy
  uint64_t sc_base;                    // global word of scratch[0], kNoScratch if unbound
  uint64_t full[kStages];              // one mbarrier per stage
  uint64_t f_src;                      // lane 0: global address of the chunk's next record
  uint32_t f_left, f_last;             // lane 0: records left in the chunk; 1 if it ends the launch
  uint32_t cnt[kStages];               // records in each stage (0 = end of work)
  uint32_t pad;
  uint32_t rk_meta, rk_rank;           // one-entry (meta -> access rank) cache, filled from chunk hints
  WarpCounts wc;
};
constexpr uint32_t kOffFull = offsetof(WarpSmem, full), kOffSrc = offsetof(WarpSmem, f_src),
                   kOffLeft = offsetof(WarpSmem, f_left), kOffLast = offsetof(WarpSmem, f_last),
                   kOffCnt = offsetof(WarpSmem, cnt),
                   kOffWc = offsetof(WarpSmem, wc), kOffScratch = offsetof(WarpSmem, scratch),
                   kOffScBase = offsetof(WarpSmem, sc_base), kOffHint = offsetof(WarpSmem, hint),
                   kOffRk = offsetof(WarpSmem, rk_meta);
constexpr uint32_t kHintFlag = 0x80000000u;   // in cnt[s]: the stage starts a chunk and carries its hint
static_assert(offsetof(WarpCounts, aff_w) == offsetof(WarpCounts, aff_u) + 4, "aff_u / aff_w adjacent");
// block layout: 8 x WarpSmem | level-1 keys (4 KB) | 256 x 56-B lane caches
// = ~66 KB: three blocks (24 warps) per SM with ~26 KB of L1
constexpr size_t kL1Off = size_t(kConsumerWarps) * sizeof(WarpSmem);
constexpr size_t kCacheOff = kL1Off + size_t(kL1MaxKeys) * 8;
constexpr size_t kAttrSmem = kCacheOff + size_t(kAttrThreads) * 56;

__device__ __forceinline__ uint8_t* attr_smem() {
  extern __shared__ __align__(128) uint8_t smem[];
  return smem;
}
// Slow-path views, rebuilt from threadIdx inside the out-of-line functions so
// that the hot loop keeps no pointers to them live.
__device__ __forceinline__ const uint64_t* slow_l1() {
  return reinterpret_cast<const uint64_t*>(attr_smem() + kL1Off);
}
__device__ __forceinline__ SlowCache* slow_cache() {
  return reinterpret_cast<SlowCache*>(attr_smem() + kCacheOff) + threadIdx.x;
}
static_assert(sizeof(SlowCache) == 56, "kAttrSmem assumes 56-B lane caches");
__device__ __forceinline__ WarpCounts* slow_counts() {
  return &reinterpret_cast<WarpSmem*>(attr_smem())[threadIdx.x >> 5].wc;
}


// small object: its whole bitmap fits the per-warp scratch (kScratchWords, below)
__device__ __forceinline__ bool small_object(uint64_t size, uint32_t shift);
__device__ __forceinline__ FastCache mirror(const SlowCache* c) {
  return FastCache{c->base, c->size, c->bm_word, c->shift, c->meta, small_object(c->size, c->shift)};
}

// Index loads (segment entries, candidates, object rows, rank table) with an
// L2 evict-last policy: the record stream is evict-first and the bitmap REDs
// evict-normal, so the lookups at chunk and burst starts keep finding the
// index in L2 instead of HBM (C5's index is 32 MB next to 1.25 GiB of shadow).
#ifndef DRGPUM_INDEX_KEEP
#define DRGPUM_INDEX_KEEP 1
#endif
__device__ __forceinline__ uint64_t evict_last_policy() {
  uint64_t p;
  asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(p));
  return p;
}
__device__ __forceinline__ uint4 ldg_keep4(const void* a) {
#if DRGPUM_INDEX_KEEP
  uint4 r;
  asm volatile("ld.global.nc.L2::cache_hint.v4.u32 {%0,%1,%2,%3}, [%4], %5;"
               : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(a), "l"(evict_last_policy()));
  return r;
#else
  return __ldg(reinterpret_cast<const uint4*>(a));
#endif
}
__device__ __forceinline__ uint32_t ldg_keep(const uint32_t* a) {
#if DRGPUM_INDEX_KEEP
  uint32_t r;
  asm volatile("ld.global.nc.L2::cache_hint.u32 %0, [%1], %2;" : "=r"(r) : "l"(a), "l"(evict_last_policy()));
  return r;
#else
  return __ldg(a);
#endif
}
__device__ __forceinline__ SegEntry ldg_seg(const SegEntry* e) {
  const uint4 v = ldg_keep4(e);
  return SegEntry{(uint64_t(v.y) << 32) | v.x, v.z, v.w};
}

// The object of segment entry e live at ts, or kNone.  Candidates are sorted
// by t_alloc with disjoint lifetimes (R5): only the last one allocated before
// ts can be live at ts (its t_free is checked by the caller).
__device__ __forceinline__ uint32_t resolve_seg(const AttrParams& p, uint32_t ref, uint32_t aux, uint32_t ts) {
  if (ref == kNone) return kNone;
  if (!(ref & kMultiBit)) return aux < ts ? ref : kNone;
  const uint32_t c0 = ref & ~kMultiBit;
  uint32_t l = c0, h = c0 + aux;
  const uint2* cand = reinterpret_cast<const uint2*>(p.cand);
  while (l < h) {
    const uint32_t mid = (l + h) >> 1;
    if (ldg_keep(&cand[mid].y) < ts) l = mid + 1; else h = mid;
  }
  return l == c0 ? kNone : ldg_keep(&cand[l - 1].x);
}

// Per-lane lookup (A2): level-1 keys (every l1_stride-th segment start) in
// shared memory, then a binary search of the segment entries in L2.
__device__ __forceinline__ uint32_t find_object(const AttrParams& p, const uint64_t* s_l1,
                                                uint64_t addr, uint32_t ts) {
  if (p.n_seg == 0 || addr < s_l1[0]) return kNone;
  uint32_t lo = 0, hi = p.n_l1;       // level 1 (shared memory): last key <= addr
  while (hi - lo > 1) {
    const uint32_t mid = (lo + hi) >> 1;
    if (s_l1[mid] <= addr) lo = mid; else hi = mid;
  }
  uint32_t a = lo * p.l1_stride;      // level 2 (L2): last segment start <= addr
  uint32_t b = min(a + p.l1_stride, p.n_seg);
  SegEntry ea = ldg_seg(p.seg + a);   // independent of the search: overlaps it
  while (b - a > 1) {
    const uint32_t mid = (a + b) >> 1;
    const SegEntry em = ldg_seg(p.seg + mid);
    if (em.start <= addr) { a = mid; ea = em; } else b = mid;
  }
  return resolve_seg(p, ea.ref, ea.aux, ts);
}

// Warp-cooperative lookup of ONE (addr, ts), uniform across the warp: every
// search level is one 32-ary round (one shared-memory or L2 load per lane and
// a ballot) instead of log2 dependent loads -- the chunk-start and burst-start
// tiles wait on this chain.
__device__ __forceinline__ uint32_t find_object_warp(const AttrParams& p, const uint64_t* s_l1, uint64_t addr,
                                                     uint32_t ts, int lane) {
  if (p.n_seg == 0 || addr < s_l1[0]) return kNone;
  // level 1: n_l1 <= 1024 keys, two rounds (s_l1[0] <= addr, so bit 0 is set)
  const uint32_t n1 = p.n_l1, step = (n1 + 31) >> 5;
  uint32_t k = uint32_t(lane) * step;
  uint32_t bal = __ballot_sync(FULL_MASK, k < n1 && s_l1[k] <= addr);
  uint32_t lo = uint32_t(31 - __clz(bal)) * step;
  k = lo + uint32_t(lane);
  bal = __ballot_sync(FULL_MASK, uint32_t(lane) < step && k < n1 && s_l1[k] <= addr);
  lo += uint32_t(31 - __clz(bal));
  // level 2: 32-ary rounds over the <= l1_stride entries after key lo
  uint32_t a = lo * p.l1_stride, w = min(p.l1_stride, p.n_seg - a);
  uint32_t ref = kNone, aux = 0;
  for (;;) {
    const uint32_t sp = (w + 31) >> 5;
    const bool in = uint32_t(lane) * sp < w;
    SegEntry e{~0ull, kNone, 0};
    if (in) e = ldg_seg(p.seg + a + uint32_t(lane) * sp);
    bal = __ballot_sync(FULL_MASK, in && e.start <= addr);   // bit 0: seg[a].start <= addr
    const int j = 31 - __clz(bal);
    a += uint32_t(j) * sp;
    if (sp == 1) {
      ref = __shfl_sync(FULL_MASK, e.ref, j);
      aux = __shfl_sync(FULL_MASK, e.aux, j);
      break;
    }
    w = min(sp, w - uint32_t(j) * sp);
  }
  if (ref == kNone) return kNone;
  if (!(ref & kMultiBit)) return aux < ts ? ref : kNone;
  // several candidates (address reuse): the last one with t_alloc < ts
  const uint2* cand = reinterpret_cast<const uint2*>(p.cand);
  const uint32_t c0 = ref & ~kMultiBit;
  uint32_t hit = kNone;
  for (uint32_t b0 = 0; b0 < aux; b0 += 32) {
    const uint32_t i = b0 + uint32_t(lane);
    const uint32_t ok = __ballot_sync(FULL_MASK, i < aux && ldg_keep(&cand[c0 + i].y) < ts);
    if (ok) hit = c0 + b0 + uint32_t(31 - __clz(ok));
    if (ok != FULL_MASK) break;   // sorted by t_alloc: the rest are later
  }
  return hit == kNone ? kNone : ldg_keep(&cand[hit].x);
}

__device__ __noinline__ void enqueue_range(RangeEntry* rq, uint32_t rq_cap, unsigned long long* ctr,
                                           uint32_t* orw, uint64_t gb0, uint64_t gb1, uint32_t& ovf) {
  const uint64_t wlo = gb0 >> 5, whi = gb1 >> 5;
  const uint64_t nch = (whi - wlo) / kRangeChunkWords + 1;
  const unsigned long long slot = atomicAdd(ctr, (unsigned long long)nch);
  for (uint64_t c = 0; c < nch; ++c) {
    const uint64_t cw0 = wlo + c * kRangeChunkWords;
    const uint64_t bl = c == 0 ? gb0 : cw0 * 32;
    const uint64_t bh = min(gb1, (cw0 + kRangeChunkWords) * 32 - 1);
    if (slot + c < rq_cap) {
      rq[slot + c] = RangeEntry{bl, bh};
    } else {  // queue full: expand this chunk in place (slow but exact)
      ovf++;
      for (uint64_t w = bl >> 5; w <= (bh >> 5); ++w) {
        uint32_t m = 0xFFFFFFFFu;
        if (w == (bl >> 5)) m &= 0xFFFFFFFFu << (bl & 31);
        if (w == (bh >> 5)) m &= 0xFFFFFFFFu >> (31 - (bh & 31));
        red_or(orw + w, m);
      }
    }
  }
}

__device__ __forceinline__ void add_counts(WarpCounts* wc, int lane, uint32_t rec, uint32_t attr,
                                           uint32_t unattr, uint32_t clip, uint32_t inval, uint32_t ovf) {
  rec = __reduce_add_sync(FULL_MASK, rec);
  attr = __reduce_add_sync(FULL_MASK, attr);
  unattr = __reduce_add_sync(FULL_MASK, unattr);
  clip = __reduce_add_sync(FULL_MASK, clip);
  inval = __reduce_add_sync(FULL_MASK, inval);
  ovf = __reduce_add_sync(FULL_MASK, ovf);
  if (lane == 0) {
    wc->rec += rec; wc->attr += attr; wc->unattr += unattr;
    wc->clip += clip; wc->inval += inval; wc->ovf += ovf;
  }
}

// ------------------------------------------------------------------ slow path
// The complete per-lane algorithm (every lane, any record).  Leaves each lane
// with c->meta = the record's meta when the record was attributed, so that
// following records of the same (object, API, rw) take the fast paths.
__device__ __noinline__ void process_slow(const AttrParams& p, uint4 r, bool present, int lane) {
  const uint64_t* s_l1 = slow_l1();
  SlowCache* c = slow_cache();
  WarpCounts* wc = slow_counts();
  const uint64_t addr = (uint64_t(r.y) << 32) | r.x;
  const uint32_t size = r.z;
  const uint32_t ts = r.w & 0x7FFFFFFFu;
  const uint32_t is_w = r.w >> 31;
  // ---- A1: validity (footnote 2: ALLOC/FREE timestamps access nothing)
  bool ok = present && size != 0 && ts < p.n_api && addr <= ~0ull - size;
  const uint32_t rank = ok ? ldg_keep(p.acc_rank + ts) : kNone;
  ok = ok && rank != kNone;
  // ---- A2: object lookup
  bool att = false;
  uint32_t clip = 0, ovf = 0;
  if (ok) {
    att = addr - c->base < c->size && ts > c->t_alloc && ts < c->t_free;
    if (!att) {
      const uint32_t o = find_object(p, s_l1, addr, ts);
      if (o != kNone) {
        const uint4* q = reinterpret_cast<const uint4*>(p.objs + o);
        const uint4 a = ldg_keep4(q), b = ldg_keep4(q + 1), d = ldg_keep4(q + 2);
        if (ts < d.y) {
          c->base = (uint64_t(a.y) << 32) | a.x;
          c->size = ((uint64_t(a.w) << 32) | a.z) - c->base;
          c->bm_word = ((uint64_t(b.y) << 32) | b.x) >> 5;
          c->hit_word = (uint64_t(b.w) << 32) | b.z;
          c->t_alloc = d.x; c->t_free = d.y; c->r_lo = d.z; c->shift = d.w;
          c->obj = o;
          att = true;
        }
      }
    }
  }
  // ---- A3: element bits
  uint64_t key0 = kNoKey, key1 = kNoKey;
  uint32_t m0 = 0, m1 = 0;
  const uint32_t obj = c->obj;
  if (att) {
    uint64_t off_end = addr - c->base + size;   // no overflow: addr+size validated
    if (off_end > c->size) { off_end = c->size; clip = 1; }
    const uint64_t gb0 = c->bm_word * 32 + ((addr - c->base) >> c->shift);
    const uint64_t gb1 = c->bm_word * 32 + ((off_end - 1) >> c->shift);
    const uint64_t w0 = gb0 >> 5, w1 = gb1 >> 5;
    if (w1 - w0 >= 2) {
      // a whole-object memcpy / memset range is expanded once per trace: the
      // first such record of the object queues it, later ones (memset then
      // memcpy-in then memcpy-out ...) set no new bit (OR is idempotent)
      const bool whole = addr == c->base && off_end == c->size;
      if (!whole || atomicOr(p.rfull + obj, 1u) == 0)
        enqueue_range(p.rq, p.rq_cap, p.ctr + p.rq_slot, p.orw, gb0, gb1, ovf);
    } else if (w1 == w0) {
      key0 = w0; m0 = bits_mask(gb0 & 31, gb1 & 31);
    } else {
      key0 = w0; m0 = 0xFFFFFFFFu << (gb0 & 31);
      key1 = w1; m1 = 0xFFFFFFFFu >> (31 - (gb1 & 31));
    }
  }
  warp_or_words(p.orw, key0, m0, lane);
  if (__any_sync(FULL_MASK, key1 != kNoKey)) warp_or_words(p.orw, key1, m1, lane);
  // ---- A4: liveness fold and hit row, one RED per run of equal objects / words
  if (__any_sync(FULL_MASK, att)) {
    bool tail;
    const uint64_t key = att ? obj : kNoKey;
    const uint32_t vmin = seg_scan(key, ts, lane, tail, OpMin());
    if (tail && att) red_min(p.first + obj, vmin);
    const uint32_t vmax = seg_scan(key, ts, lane, tail, OpMax());
    if (tail && att) red_max(p.last + obj, vmax);
    uint64_t hkey = kNoKey;
    uint32_t hm = 0;
    if (att) {
      const uint32_t hb = 2 * (rank - c->r_lo) + is_w;
      hkey = c->hit_word + (hb >> 5);
      hm = 1u << (hb & 31);
    }
    warp_or_words(p.orw, hkey, hm, lane);
  }
  c->meta = att ? r.w : kNever;
  add_counts(wc, lane, present, att, ok && !att, clip, present && !ok, ovf);
}

// ------------------------------------------------------------------ fast path
// Preconditions (checked by the caller): every lane's cache holds the SAME
// object (< 4 GiB) and the same (API, rw) whose first/last/hit work is done,
// and every lane's record lies inside that object, unclipped, <= 2 words.
// e0/e1 are element indices relative to the object; bm_word its first word.
// Only the bitmap OR remains.
// OR the element range [e0, e1] (at most two words) of an object's bitmap.
// OR is idempotent, so records sharing a word need no warp-level merge; the
// L2 atomic units have the headroom (ncu: ~15% busy), the issue slots do not.
// Elements [e0, e0 + len] (len < 32) as the masks of word e0 >> 5 (lo) and
// of the next word (hi, 0 when the range stays in one word): len + 1 ones
// shifted left by e0 % 32 across the 64-bit word pair (two funnel shifts,
// which take the shift modulo 32).
__device__ __forceinline__ void range_masks(uint32_t e0, uint32_t len, uint32_t& lo, uint32_t& hi) {
  const uint32_t m = (2u << len) - 1u;   // len = 31: 2 << 31 = 0 in 32 bits -> all ones
  lo = __funnelshift_l(0u, m, e0);
  hi = __funnelshift_l(m, 0u, e0);
}
__device__ __forceinline__ void red_range(uint32_t* orw, uint64_t bm_word, uint32_t e0, uint32_t len) {
  uint32_t lo, hi;
  range_masks(e0, len, lo, hi);
  uint32_t* a = orw + bm_word + (e0 >> 5);
  red_or(a, lo);
  if (hi) red_or(a + 1, hi);
}
__device__ __forceinline__ void red_record(uint32_t* orw, uint64_t bm_word, uint32_t e0, uint32_t e1) {
  red_range(orw, bm_word, e0, e1 - e0);
}

// --- small-object scratch (warp-uniform calls)
__device__ __forceinline__ bool small_object(uint64_t size, uint32_t shift) {
  return kScratchWords > 0 && size <= (uint64_t(kScratchWords) * 32) << shift;
}
__device__ __forceinline__ bool scratch_ok(const FastCache& c) { return c.sc; }
__device__ __forceinline__ void red_shared_or(uint32_t a, uint32_t v) {
  asm volatile("red.shared.or.b32 [%0], %1;" ::"r"(a), "r"(v) : "memory");
}
// OR every nonzero scratch word into the global bitmap at sc_base and clear it
__device__ __noinline__ void scratch_flush(uint32_t wsm, uint32_t* orw, uint64_t sc_base, int lane) {
  __syncwarp();   // every lane's shared REDs are done
#pragma unroll
  for (uint32_t i = lane; i < kScratchWords; i += 32) {
    const uint32_t a = wsm + kOffScratch + 4 * i;
    uint32_t v;
    asm volatile("ld.shared.u32 %0, [%1];" : "=r"(v) : "r"(a) : "memory");
    if (v) {
      red_or(orw + sc_base + i, v);
      sts32(a, 0);
    }
  }
  __syncwarp();
}
// bind the scratch to the object whose bitmap starts at bm_word (flushing the
// previous object's bits)
__device__ __forceinline__ void scratch_bind(uint32_t wsm, uint32_t* orw, uint64_t bm_word, int lane) {
  const uint64_t cur = lds64(wsm + kOffScBase);
  if (cur == bm_word) return;   // warp-uniform
  if (cur != kNoScratch) scratch_flush(wsm, orw, cur, lane);
  else __syncwarp();            // every lane has read cur before lane 0 overwrites it
  if (lane == 0) sts64(wsm + kOffScBase, bm_word);
  __syncwarp();
}
__device__ __forceinline__ void scratch_range(uint32_t wsm, uint32_t e0, uint32_t len) {
  uint32_t lo, hi;
  range_masks(e0, len, lo, hi);
  const uint32_t a = wsm + kOffScratch + 4 * (e0 >> 5);
  red_shared_or(a, lo);
  if (hi) red_shared_or(a + 4, hi);
}
__device__ __forceinline__ void scratch_record(uint32_t wsm, uint32_t e0, uint32_t e1) {
  scratch_range(wsm, e0, e1 - e0);
}

__device__ __forceinline__ void fast_or(uint32_t* orw, uint64_t bm_word, uint32_t e0, uint32_t e1, int lane) {
  // contiguous union: intervals chain (start within or right after the
  // previous interval, monotone ends) -> union = [e0 of lane 0, e1 of lane 31]
  const uint32_t pe0 = __shfl_up_sync(FULL_MASK, e0, 1);
  const uint32_t pe1 = __shfl_up_sync(FULL_MASK, e1, 1);
  const bool chain = lane == 0 || (e0 >= pe0 && e0 <= pe1 + 1 && e1 >= pe1);
  if (__all_sync(FULL_MASK, chain)) {
    const uint32_t lo = __shfl_sync(FULL_MASK, e0, 0);
    const uint32_t hi = __shfl_sync(FULL_MASK, e1, 31);
    const uint32_t wlo = lo >> 5, nw = (hi >> 5) - wlo;   // words wlo .. wlo+nw
    uint32_t* base = orw + bm_word + wlo;
    for (uint32_t w = lane; w <= nw; w += 32) {
      uint32_t m = 0xFFFFFFFFu;
      if (w == 0) m &= 0xFFFFFFFFu << (lo & 31);
      if (w == nw) m &= 0xFFFFFFFFu >> (31 - (hi & 31));
      red_or(base + w, m);
    }
    return;
  }
  red_record(orw, bm_word, e0, e1);   // irregular: each record ORs its own word(s)
}
// fast_or for the warp's cached object c: irregular tiles of a small object
// go through the scratch
__device__ __forceinline__ void fast_or_c(uint32_t wsm, uint32_t* orw, const FastCache& c, uint32_t e0,
                                          uint32_t e1, int lane) {
  if (scratch_ok(c)) {
#if DRGPUM_UNION_SCRATCH
    scratch_bind(wsm, orw, c.bm_word, lane);   // chained or not: the scratch
    scratch_record(wsm, e0, e1);
    return;
#else
    const uint32_t pe0 = __shfl_up_sync(FULL_MASK, e0, 1);
    const uint32_t pe1 = __shfl_up_sync(FULL_MASK, e1, 1);
    const bool chain = lane == 0 || (e0 >= pe0 && e0 <= pe1 + 1 && e1 >= pe1);
    if (!__all_sync(FULL_MASK, chain)) {
      scratch_bind(wsm, orw, c.bm_word, lane);
      scratch_record(wsm, e0, e1);
      return;
    }
#endif
  }
#if DRGPUM_WINDOW
  else {   // a large object's irregular tile within < 64 words: scratch window
    const uint32_t pe0 = __shfl_up_sync(FULL_MASK, e0, 1);
    const uint32_t pe1 = __shfl_up_sync(FULL_MASK, e1, 1);
    const bool chain = lane == 0 || (e0 >= pe0 && e0 <= pe1 + 1 && e1 >= pe1);
    if (!__all_sync(FULL_MASK, chain)) {
      const uint32_t lo_w = __reduce_min_sync(FULL_MASK, e0) >> 5, hi_w = __reduce_max_sync(FULL_MASK, e1) >> 5;
      if (kScratchWords >= 128 && hi_w - lo_w < 64) {
        const uint32_t wb = lo_w & ~63u;
        scratch_bind(wsm, orw, c.bm_word + wb, lane);
        scratch_record(wsm, e0 - 32 * wb, e1 - 32 * wb);
        return;
      }
      red_record(orw, c.bm_word, e0, e1);
      return;
    }
  }
#endif
  fast_or(orw, c.bm_word, e0, e1, lane);
}

// Affine tier: the warp's 128 consecutive records (4 tiles, lane l holds
// records l, 32+l, 64+l, 96+l) are one constant-stride run of one size and one
// (API, rw) inside the warp's cached object: addr_j = a0 + j*st.  This is
// what warp-coalesced instrumentation emits for a[i] sweeps and strided
// loops.  Validity, liveness, first/last and the hit bit are then settled by
// the cache; when consecutive records overlap or touch adjacent elements
// (st <= size or st <= elem_size) the union is ONE element range, written
// with one RED.OR per word; otherwise each record ORs its own word(s).
// Returns false (no side effect) when the precondition does not hold.
__device__ __forceinline__ int try_affine(const uint4 (&r)[kTilesPerWarp], const FastCache& c,
                                           uint32_t* orw, uint32_t wsm, int lane) {
  // predicted record j = 32k + lane: {lo(a0) + j*st, hi(a0), sz, meta}; the
  // mismatch bits of all four words of all records are ORed with 3-input
  // LOP3s (about 5 instructions per record)
  const uint32_t a0lo = __shfl_sync(FULL_MASK, r[0].x, 0);
  const uint32_t st32 = __shfl_sync(FULL_MASK, r[0].x, 1) - a0lo;
  uint32_t exp = a0lo + uint32_t(lane) * st32;
  // the first tile's low address words first: most stages that are not
  // affine (wrapping strided sweeps, gathers) fail here, before the rest
  if (!__all_sync(FULL_MASK, r[0].x == exp)) return 0;
  const uint32_t a0hi = __shfl_sync(FULL_MASK, r[0].y, 0);
  const uint32_t sz = __shfl_sync(FULL_MASK, r[0].z, 0);
  uint32_t bad = (r[0].y ^ a0hi) | (r[0].z ^ sz) | (r[0].w ^ c.meta);
#pragma unroll
  for (int k = 1; k < kTilesPerWarp; ++k) {
    exp += 32u * st32;
    bad |= (r[k].x ^ exp) | (r[k].y ^ a0hi);
    bad |= (r[k].z ^ sz) | (r[k].w ^ c.meta);
  }
  if (!__all_sync(FULL_MASK, bad == 0)) return 0;
  // uniform from here on: every lane holds the same values
  constexpr uint32_t kN = 32 * kTilesPerWarp;
  // the prediction is exact only if the low word never wrapped: then record j
  // is at a0 + j*st in 64 bits
  const uint64_t a0 = (uint64_t(a0hi) << 32) | a0lo;
  if (st32 == 0 || sz == 0 || uint64_t(a0lo) + uint64_t(kN - 1) * st32 + sz > (1ull << 32)) return 0;
  const uint64_t off0 = a0 - c.base;
  if (off0 >= c.size) return 0;
  const uint64_t off_end = off0 + uint64_t(kN - 1) * st32 + sz;     // one past the last byte
  if (off_end > c.size) return 0;
  const uint32_t o0 = uint32_t(off0);                                // c.size < 2^32 (uni)
  if (st32 <= sz || st32 <= (1u << c.shift)) {
    const uint32_t lo = o0 >> c.shift, hi = uint32_t(off_end - 1) >> c.shift;
    const uint32_t wlo = lo >> 5, nw = (hi >> 5) - wlo;
#if DRGPUM_UNION_SCRATCH
    // a small object's union goes to the scratch: a sweep that wraps around
    // the object (C5's 8 KiB objects, C3's activations) re-ORs the same
    // words every pass, in shared memory instead of as global RED sectors
    if (scratch_ok(c)) {
      scratch_bind(wsm, orw, c.bm_word, lane);
      for (uint32_t w = lane; w <= nw; w += 32) {
        uint32_t m = 0xFFFFFFFFu;
        if (w == 0) m &= 0xFFFFFFFFu << (lo & 31);
        if (w == nw) m &= 0xFFFFFFFFu >> (31 - (hi & 31));
        red_shared_or(wsm + kOffScratch + 4 * (wlo + w), m);
      }
      return 1;
    }
#endif
    uint32_t* base = orw + c.bm_word + wlo;
    for (uint32_t w = lane; w <= nw; w += 32) {
      uint32_t m = 0xFFFFFFFFu;
      if (w == 0) m &= 0xFFFFFFFFu << (lo & 31);
      if (w == nw) m &= 0xFFFFFFFFu >> (31 - (hi & 31));
      red_or(base + w, m);
    }
    return 1;
  }
  // records of up to 31 elements after the first (range_masks): wider ones take the tile path
  if (((sz - 1) >> c.shift) >= 31) return 0;
  // not one range: every record ORs its own word(s) (offsets in 32 bits),
  // through the scratch for a small object
  uint32_t off = o0 + uint32_t(lane) * st32;
  if (scratch_ok(c)) {
    scratch_bind(wsm, orw, c.bm_word, lane);
#pragma unroll
    for (int k = 0; k < kTilesPerWarp; ++k) {
      scratch_record(wsm, off >> c.shift, (off + sz - 1) >> c.shift);
      off += 32u * st32;
    }
    return 2;
  }
#if DRGPUM_WINDOW
  // a large object's strided sweep whose 128 records span < 64 words: OR
  // them into a 128-word scratch window of the object (consecutive stages of
  // a sweep with stride < 16 elements share it), flushed when the window moves
  {
    const uint32_t lo_w = (o0 >> c.shift) >> 5;
    const uint32_t hi_w = (uint32_t(off_end - 1) >> c.shift) >> 5;
    if (kScratchWords >= 128 && hi_w - lo_w < 64) {
      const uint32_t wb = lo_w & ~63u;
      scratch_bind(wsm, orw, c.bm_word + wb, lane);
#pragma unroll
      for (int k = 0; k < kTilesPerWarp; ++k) {
        scratch_record(wsm, (off >> c.shift) - 32 * wb, ((off + sz - 1) >> c.shift) - 32 * wb);
        off += 32u * st32;
      }
      return 2;
    }
  }
#endif
#pragma unroll
  for (int k = 0; k < kTilesPerWarp; ++k) {
    red_record(orw, c.bm_word, off >> c.shift, (off + sz - 1) >> c.shift);
    off += 32u * st32;
  }
  return 2;
}

// In-object tier: the warp's 128 records all carry the cached (API, rw) and
// start inside the cached object (< 4 GiB), <= 32 elements each after the
// clip at the object's end, in any
// order (random gathers, strided sweeps that wrap).  Each record ORs its own
// word(s): no warp analysis, OR is idempotent.  Returns false without side
// effects otherwise.
__device__ __forceinline__ bool try_in_object(const uint4 (&r)[kTilesPerWarp], const FastCache& c,
                                              uint32_t* orw, uint32_t wsm, int lane) {
  const uint32_t osz = uint32_t(c.size);
  uint32_t e0[kTilesPerWarp], ln[kTilesPerWarp];
  bool ok = true;
  uint32_t nclip = 0;
#pragma unroll
  for (int k = 0; k < kTilesPerWarp; ++k) {
    // off < c.size (< 2^32 here) also bounds the high word and off32 < osz
    const uint64_t off = ((uint64_t(r[k].y) << 32) | r[k].x) - c.base;
    const uint32_t off32 = uint32_t(off), room = osz - off32;
    const uint32_t sz = min(r[k].z, room);   // clipped at the object's end (R3)
    nclip += r[k].z > room;
    e0[k] = off32 >> c.shift;
    ln[k] = ((off32 + sz - 1) >> c.shift) - e0[k];
    ok = ok && off < c.size && r[k].w == c.meta && r[k].z != 0 && ln[k] < 32;
  }
  if (!__all_sync(FULL_MASK, ok)) return false;
  if (__any_sync(FULL_MASK, nclip != 0)) {
    nclip = __reduce_add_sync(FULL_MASK, nclip);
    if (lane == 0) red_shared_add<kOffWc + offsetof(WarpCounts, clip)>(wsm, nclip);
  }
  if (scratch_ok(c)) {
    scratch_bind(wsm, orw, c.bm_word, lane);
#pragma unroll
    for (int k = 0; k < kTilesPerWarp; ++k) scratch_range(wsm, e0[k], ln[k]);
    return true;
  }
#if DRGPUM_WINDOW
  {   // the 128 records of a large object within < 64 words: scratch window
    uint32_t lo = e0[0], hi = e0[0] + ln[0];
#pragma unroll
    for (int k = 1; k < kTilesPerWarp; ++k) { lo = min(lo, e0[k]); hi = max(hi, e0[k] + ln[k]); }
    const uint32_t lo_w = __reduce_min_sync(FULL_MASK, lo) >> 5, hi_w = __reduce_max_sync(FULL_MASK, hi) >> 5;
    if (kScratchWords >= 128 && hi_w - lo_w < 64) {
      const uint32_t wb = lo_w & ~63u;
      scratch_bind(wsm, orw, c.bm_word + wb, lane);
#pragma unroll
      for (int k = 0; k < kTilesPerWarp; ++k) scratch_range(wsm, e0[k] - 32 * wb, ln[k]);
      return true;
    }
  }
#endif
#pragma unroll
  for (int k = 0; k < kTilesPerWarp; ++k) red_range(orw, c.bm_word, e0[k], ln[k]);
  return true;
}

// Warp-uniform slow path: all 32 records share one (API, rw) and land in one
// object (the first tile of every burst).  One lane resolves the object and
// folds first/last/hit once for the warp; the lanes adopt the object into
// their caches.  Returns false (no side effect) when the precondition fails.
__device__ __noinline__ bool try_uniform_slow(const AttrParams& p, uint4 r, bool present, int lane) {
  const uint64_t* s_l1 = slow_l1();
  SlowCache* c = slow_cache();
  WarpCounts* wc = slow_counts();
  const uint32_t meta = r.w;
  const uint32_t meta0 = __shfl_sync(FULL_MASK, meta, 0);   // all lanes: never inside && / ||
  if (!__all_sync(FULL_MASK, present && meta == meta0)) return false;
  const uint32_t ts = meta & 0x7FFFFFFFu, is_w = meta >> 31;
  if (ts >= p.n_api) return false;
  // the access rank: from the warp's one-entry cache (a chunk hint's first
  // record) or loaded; checked after the search, whose latency it overlaps
  const uint32_t wsm = smem_u32(attr_smem()) + (threadIdx.x >> 5) * uint32_t(sizeof(WarpSmem));
  const uint32_t rank = lds32<kOffRk>(wsm) == meta ? lds32<kOffRk + 4>(wsm) : ldg_keep(p.acc_rank + ts);
  const uint64_t addr = (uint64_t(r.y) << 32) | r.x;
  const uint64_t addr0 = __shfl_sync(FULL_MASK, addr, 0);
  uint64_t base, osz, bm_word, hit_word;
  uint32_t o, t_alloc, t_free, r_lo, shift;
  if (__all_sync(FULL_MASK, addr0 - c->base < c->size && ts > c->t_alloc && ts < c->t_free)) {
    // every lane's cached object contains addr0 and is live at ts: it is THE
    // object (R5: live objects never overlap) -- no search (chunk starts
    // with a hint, a new API on the same object)
    base = c->base; osz = c->size; bm_word = c->bm_word; hit_word = c->hit_word;
    o = c->obj; t_alloc = c->t_alloc; t_free = c->t_free; r_lo = c->r_lo; shift = c->shift;
  } else {
    o = find_object_warp(p, s_l1, addr0, ts, lane);
    if (o == kNone) return false;
    const uint4* q = reinterpret_cast<const uint4*>(p.objs + o);
    const uint4 a = ldg_keep4(q), b = ldg_keep4(q + 1), d = ldg_keep4(q + 2);
    base = (uint64_t(a.y) << 32) | a.x;
    osz = ((uint64_t(a.w) << 32) | a.z) - base;
    bm_word = ((uint64_t(b.y) << 32) | b.x) >> 5;
    hit_word = (uint64_t(b.w) << 32) | b.z;
    t_alloc = d.x; t_free = d.y; r_lo = d.z; shift = d.w;
  }
  if (rank == kNone || ts >= t_free) return false;
  if (osz > 0xFFFFFFFFull) return false;
  const uint64_t off = addr - base;
  const uint32_t size = r.z;
  const uint32_t off32 = uint32_t(off), e0 = off32 >> shift, e1 = (off32 + size - 1) >> shift;
  const bool ok = off < osz && size != 0 && size <= uint32_t(osz) - off32 && e1 - e0 < 32;
  if (!__all_sync(FULL_MASK, ok)) return false;
  c->base = base; c->size = osz;
  c->bm_word = bm_word;
  c->hit_word = hit_word;
  c->t_alloc = t_alloc; c->t_free = t_free; c->r_lo = r_lo; c->shift = shift; c->obj = o;
  c->meta = meta;
  if (lane == 0) {
    const uint32_t hb = 2 * (rank - r_lo) + is_w;
    red_min(p.first + o, ts);
    red_max(p.last + o, ts);
    red_or(p.orw + c->hit_word + (hb >> 5), 1u << (hb & 31));
    wc->rec += 32;
    wc->attr += 32;
  }
  fast_or(p.orw, c->bm_word, e0, e1, lane);
  return true;
}

__global__ void __launch_bounds__(kAttrThreads, DRGPUM_MINBLOCKS) attribute_kernel(const __grid_constant__ AttrParams p) {
  extern __shared__ __align__(128) uint8_t smem[];
  const int lane = threadIdx.x & 31;
  // this warp's region (shared-window address): ring | barriers | fetch state | counters
  const uint32_t wsm = smem_u32(smem) + (threadIdx.x >> 5) * uint32_t(sizeof(WarpSmem));

  // Work distribution: warps take contiguous chunks (chunk_start) of records
  // from a global cursor (dynamic, so slow warps do not set the kernel's end).
  // Only lane 0 touches the fetch state (shared memory, plus the prefetched
  // ticket of the next chunk in a register).
  const uint32_t n_warps = gridDim.x * (kAttrThreads / 32);
  // lane 0: ticket of the next chunk, taken two stages ahead (static: its own range first)
  uint32_t f_next = kStatic ? blockIdx.x * (kAttrThreads / 32) + (threadIdx.x >> 5) : kNone;
  auto ticket = [&]() { return take_ticket(&p.ctr[C_WORK]) + (kStatic ? n_warps : 0u); };
#if DRGPUM_FETCH_V2
  auto fetch = [&](int s) {   // lane 0: fill slot s with the next <= 128 records, or mark the end
    // per stage: records left (u32) and the next record's address (u64) --
    // a new chunk only every 64 stages; no 64-bit position arithmetic
    uint32_t left = lds32<kOffLeft>(wsm);
    uint64_t src;
    uint32_t hk = kNone;   // the chunk whose first stage this is (hint index)
    if (left == 0) {
      uint64_t lo, hi;
      do {   // skip empty chunks (only possible at the end or in a tiny static part)
        const uint32_t kc = f_next == kNone ? ticket() : f_next;
        hk = kc;
        f_next = kNone;
        lo = min(chunk_start(kc, p, n_warps), p.n);
        hi = min(chunk_start(uint64_t(kc) + 1, p, n_warps), p.n);
      } while (lo == hi && lo < p.n);
      if (lo >= p.n) lo = hi = p.n;
      left = uint32_t(hi - lo);
      src = reinterpret_cast<uint64_t>(p.recs + lo);
      sts32(wsm + kOffLast, hi >= p.n ? 1u : 0u);
    } else {
      src = lds64(wsm + kOffSrc);
    }
    const uint32_t cnt = min(uint32_t(kWarpRecords), left);
    const bool hinted = cnt && hk < p.hint_cap;
    sts32(wsm + kOffCnt + 4 * s, cnt | (hinted ? kHintFlag : 0u));
    const uint32_t bar = wsm + kOffFull + 8 * s;
    if (cnt) {
      mbar_arrive_expect_tx(bar, cnt * 16 + (hinted ? uint32_t(sizeof(ChunkHint)) : 0u));
      tma_load_1d(wsm + s * (kWarpRecords * 16), reinterpret_cast<const void*>(src), cnt * 16, bar,
                  evict_first_policy());
      if (hinted)   // the chunk's hint rides on the same barrier
        tma_load_1d(wsm + kOffHint + s * uint32_t(sizeof(ChunkHint)), p.hints + hk, uint32_t(sizeof(ChunkHint)), bar,
                    evict_first_policy());
      sts64(wsm + kOffSrc, src + 16ull * cnt);
      left -= cnt;
      sts32(wsm + kOffLeft, left);
      // the next chunk's ticket is taken when this one has at most two stages
      // left: its latency hides behind them, and no warp holds a reservation
      // long enough to unbalance the end of the launch
      if (left <= DRGPUM_TICKET_AHEAD * kWarpRecords && f_next == kNone && !lds32<kOffLast>(wsm))
        f_next = ticket();
    } else {
      mbar_arrive(bar);   // end of work: complete the phase with cnt = 0
    }
  };

#else
  // A/B reference: 64-bit [f_pos, f_hi) kept in the f_src / (f_left, f_last) words
  auto fetch = [&](int s) {   // lane 0: fill slot s with the next <= 128 records, or mark the end
    uint64_t f_pos = lds64(wsm + kOffSrc), f_hi = lds64(wsm + kOffLeft);
    if (f_pos == f_hi) {
      do {   // skip empty chunks (only possible at the end or in a tiny static part)
        const uint32_t kc = f_next == kNone ? ticket() : f_next;
        f_next = kNone;
        f_pos = min(chunk_start(kc, p, n_warps), p.n);
        f_hi = min(chunk_start(uint64_t(kc) + 1, p, n_warps), p.n);
      } while (f_pos == f_hi && f_pos < p.n);
      if (f_pos >= p.n) f_pos = f_hi = p.n;
      sts64(wsm + kOffLeft, f_hi);
    }
    const uint32_t cnt = uint32_t(min(uint64_t(kWarpRecords), f_hi - f_pos));
    sts32(wsm + kOffCnt + 4 * s, cnt);
    const uint32_t bar = wsm + kOffFull + 8 * s;
    if (cnt) {
      mbar_arrive_expect_tx(bar, cnt * 16);
      tma_load_1d(wsm + s * (kWarpRecords * 16), p.recs + f_pos, cnt * 16, bar, evict_first_policy());
      f_pos += cnt;
      sts64(wsm + kOffSrc, f_pos);
      // the next chunk's ticket is taken when this one has at most two stages
      // left: its latency hides behind them, and no warp holds a reservation
      // long enough to unbalance the end of the launch
      if (f_next == kNone && f_hi - f_pos <= 2 * kWarpRecords && f_hi < p.n)
        f_next = ticket();
    } else {
      mbar_arrive(bar);   // end of work: complete the phase with cnt = 0
    }
  };

#endif
  for (uint32_t i = lane; i < kScratchWords; i += 32) sts32(wsm + kOffScratch + 4 * i, 0);
  SlowCache* my = slow_cache();
  my->base = 0; my->size = 0; my->bm_word = 0; my->hit_word = 0;
  my->t_alloc = 0; my->t_free = 0; my->r_lo = 0; my->shift = 0; my->obj = kNone; my->meta = kNever;
  if (lane == 0) {
    *slow_counts() = WarpCounts{0, 0, 0, 0, 0, 0, 0, 0, 0, 0};
    sts64(wsm + kOffSrc, 0);
    sts32(wsm + kOffLeft, 0);
    sts32(wsm + kOffLast, 0);
    sts64(wsm + kOffScBase, kNoScratch);
    sts32(wsm + kOffRk, kNever);
    for (int s = 0; s < kStages; ++s) mbar_init(wsm + kOffFull + 8 * s, 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    for (int s = 0; s < kStages; ++s) fetch(s);
  }
  {
    uint64_t* s_l1 = reinterpret_cast<uint64_t*>(smem + kL1Off);
    for (uint32_t i = threadIdx.x; i < p.n_l1; i += blockDim.x) s_l1[i] = p.l1[i];
  }
  __syncthreads();

  FastCache c = mirror(my);
  uint32_t fast_rec = 0;
  bool uni = false;  // warp-uniform: all lanes cache one object (< 4 GiB) and one (API, rw)
  for (uint32_t st = 0;; ++st) {
    const int s = int(st % kStages);
    mbar_wait<kOffFull>(wsm + 8 * s, (st / kStages) & 1);
    uint32_t cnt = lds32<kOffCnt>(wsm + 4 * s);
    if (cnt == 0) break;                                   // warp-uniform
    if (cnt & kHintFlag) {
      // a new chunk: every lane's cache takes the object of its first record
      // (resolved by chunk_hint_kernel), with no API folded yet (meta =
      // NEVER), so the first tile's uniform slow path finds the object in the
      // cache instead of searching the index
      cnt &= ~kHintFlag;
      const uint32_t hb = wsm + kOffHint + s * uint32_t(sizeof(ChunkHint));
      const uint4 h0 = lds128(hb), h1 = lds128(hb + 16), h2 = lds128(hb + 32), h3 = lds128(hb + 48);
      if (h3.x != kNone) {
        SlowCache* my = slow_cache();
        my->base = (uint64_t(h0.y) << 32) | h0.x;
        my->size = ((uint64_t(h0.w) << 32) | h0.z) - my->base;
        my->bm_word = ((uint64_t(h1.y) << 32) | h1.x) >> 5;
        my->hit_word = (uint64_t(h1.w) << 32) | h1.z;
        my->t_alloc = h2.x; my->t_free = h2.y; my->r_lo = h2.z; my->shift = h2.w; my->obj = h3.x;
        my->meta = kNever;
        c = mirror(my);
        uni = false;
        if (lane == 0) { sts32(wsm + kOffRk, h3.y); sts32(wsm + kOffRk + 4, h3.z); }
      }
    }
    const int ntiles = int((cnt + 31) / 32);
    // copy the stage to registers (lane l: records l, 32+l, 64+l, 96+l) and refill the slot
    const uint32_t sbuf = wsm + s * (kWarpRecords * 16) + lane * 16;
    uint4 r4[kTilesPerWarp];
    if (cnt == kWarpRecords) {                             // full stage (all but a chunk's tail)
#pragma unroll
      for (int t = 0; t < kTilesPerWarp; ++t) r4[t] = lds128(sbuf + t * 512);
    } else {
#pragma unroll
      for (int t = 0; t < kTilesPerWarp; ++t)
        r4[t] = t * 32 + lane < cnt ? lds128(sbuf + t * 512) : make_uint4(0, 0, 0, 0);
    }
    // The vote consumes every lane's loaded registers, so all of this warp's
    // reads of the slot have completed before lane 0 refills it.  This is a
    // write-after-read across proxies with the reads already retired, so no
    // proxy fence (as a consumer release before a TMA refill; a memory fence
    // would also wait for this lane's outstanding global REDs).
    uint32_t dep = 0;
#pragma unroll
    for (int t = 0; t < kTilesPerWarp; ++t) dep ^= r4[t].x;   // one register per LDS.128 suffices
    const bool never = __any_sync(FULL_MASK, dep == 0x9E3779B9u && lane == 32);
    if (lane == 0 && !never) fetch(s);
    __syncwarp();
    if (uni && ntiles == kTilesPerWarp) {
      const int how = try_affine(r4, c, p.orw, wsm, lane);
      if (how) {
        fast_rec += kTilesPerWarp;
        if (lane == 0) red_shared_add<kOffWc + offsetof(WarpCounts, aff_u)>(wsm + (how == 1 ? 0 : 4), kTilesPerWarp);
        continue;
      }
      if (try_in_object(r4, c, p.orw, wsm, lane)) {
        fast_rec += kTilesPerWarp;
        continue;
      }
    }
#pragma unroll 1
    for (int t = 0; t < ntiles; ++t) {
      const bool present = t * 32 + lane < cnt;
      uint4 r = r4[0];                       // register select, no local-memory indexing
#pragma unroll
      for (int j = 1; j < kTilesPerWarp; ++j) if (t == j) r = r4[j];
      if (uni) {
        // fast check in 32-bit object-relative arithmetic
        const uint64_t off = ((uint64_t(r.y) << 32) | r.x) - c.base;
        const uint32_t off32 = uint32_t(off), size = r.z, osz = uint32_t(c.size), room = osz - off32;
        const bool clip = size > room;   // runs past the object's end: clipped there (R3)
        const uint32_t e0 = off32 >> c.shift;
        const uint32_t e1 = (off32 + (clip ? room : size) - 1) >> c.shift;
        const bool ok = present && r.w == c.meta && (off >> 32) == 0 && off32 < osz &&
                        size != 0 && e1 - e0 < 32;
        if (__all_sync(FULL_MASK, ok)) {
          const uint32_t nclip = __popc(__ballot_sync(FULL_MASK, clip));
          if (nclip && lane == 0) red_shared_add<kOffWc + offsetof(WarpCounts, clip)>(wsm, nclip);
          fast_or_c(wsm, p.orw, c, e0, e1, lane);
          ++fast_rec;
          continue;
        }
      }
      if (!try_uniform_slow(p, r, present, lane)) process_slow(p, r, present, lane);
      if (lane == 0) red_shared_add<kOffWc + offsetof(WarpCounts, slow)>(wsm, 1);
      SlowCache* my = slow_cache();
      c = mirror(my);
      const uint32_t m0 = __shfl_sync(FULL_MASK, c.meta, 0);
      const uint32_t o0 = __shfl_sync(FULL_MASK, my->obj, 0);
      uni = __all_sync(FULL_MASK, c.meta == m0 && my->obj == o0 && m0 != kNever && c.size <= 0xFFFFFFFFull);
    }
  }
  if (kScratchWords > 0) {   // the small-object scratch's last bits
    const uint64_t sc = lds64(wsm + kOffScBase);
    if (sc != kNoScratch) scratch_flush(wsm, p.orw, sc, lane);
  }
  // A5: counters -- fast-path records per lane plus the warp's slow-path sums
  const uint32_t fr = __reduce_add_sync(FULL_MASK, fast_rec);
  __syncwarp();
  if (lane == 0) {
    const WarpCounts* wc = slow_counts();
    const uint32_t v[6] = {wc->rec + fr, wc->attr + fr, wc->unattr, wc->clip, wc->inval, wc->ovf};
    const int slot[6] = {C_RECORDS, C_ATTRIBUTED, C_UNATTRIBUTED, C_CLIPPED, C_INVALID, C_RQ_OVERFLOW};
#pragma unroll
    for (int i = 0; i < 6; ++i)
      if (v[i]) atomicAdd(&p.ctr[slot[i]], (unsigned long long)v[i]);
    atomicAdd(&p.ctr[C_TILES_AFFINE_UNION], (unsigned long long)wc->aff_u);
    atomicAdd(&p.ctr[C_TILES_AFFINE_WORDS], (unsigned long long)wc->aff_w);
    // fast tiles (in-object tier, tile fast path) = fast-path tiles - affine tiles
    atomicAdd(&p.ctr[C_TILES_FAST], (unsigned long long)(fr / 32 - wc->aff_u - wc->aff_w));
    atomicAdd(&p.ctr[C_TILES_SLOW], (unsigned long long)wc->slow);
  }
}

// B2: expand queued ranges: one warp per <= kRangeChunkWords-word entry;
// interior words get a plain all-ones store (idempotent with concurrent ORs),
// edge words a RED.OR.
// The counters the attribution kernel consumed are re-armed here for the next
// call (no memset nodes between calls): the work cursor, and the queue count
// of the OTHER parity -- this call's count is still being read by every block.
__global__ void __launch_bounds__(256) range_expand_kernel(const RangeEntry* rq,
    unsigned long long* ctr, uint32_t slot, uint32_t cap, uint32_t* orw) {
  if (blockIdx.x == 0 && threadIdx.x == 0) {
    ctr[C_WORK] = 0;
    ctr[slot == C_RQ_COUNT ? C_RQ_COUNT_ALT : C_RQ_COUNT] = 0;
  }
  const unsigned long long cnt_raw = ctr[slot];
  const uint64_t cnt = cnt_raw < cap ? cnt_raw : cap;
  const int lane = threadIdx.x & 31;
  const uint64_t gwarp = (uint64_t(blockIdx.x) * blockDim.x + threadIdx.x) >> 5;
  const uint64_t nwarps = (uint64_t(gridDim.x) * blockDim.x) >> 5;
  for (uint64_t e = gwarp; e < cnt; e += nwarps) {
    const RangeEntry r = rq[e];
    const uint64_t w0 = r.bit_lo >> 5, w1 = r.bit_hi >> 5;
    // edge words: masked RED; interior: all-ones, 16-B stores on the
    // 4-word-aligned middle and scalar stores around it
    if (lane == 0) red_or(orw + w0, w0 == w1 ? (0xFFFFFFFFu << (r.bit_lo & 31)) &
                                                 (0xFFFFFFFFu >> (31 - (r.bit_hi & 31)))
                                               : 0xFFFFFFFFu << (r.bit_lo & 31));
    if (lane == 1 && w1 != w0) red_or(orw + w1, 0xFFFFFFFFu >> (31 - (r.bit_hi & 31)));
    if (w1 <= w0 + 1) continue;
    const uint64_t i0 = w0 + 1, i1 = w1;                 // interior [i0, i1)
    const uint64_t a0 = (i0 + 3) & ~3ull, a1 = i1 & ~3ull;
    if (a0 >= a1) {
      for (uint64_t w = i0 + lane; w < i1; w += 32) orw[w] = 0xFFFFFFFFu;
      continue;
    }
    if (i0 + lane < a0) orw[i0 + lane] = 0xFFFFFFFFu;
    if (a1 + lane < i1) orw[a1 + lane] = 0xFFFFFFFFu;
    uint4* v = reinterpret_cast<uint4*>(orw + a0);
    const uint64_t nv = (a1 - a0) >> 2;
    for (uint64_t k = lane; k < nv; k += 32) v[k] = make_uint4(~0u, ~0u, ~0u, ~0u);
  }
}

// Chunk-start hints: thread k resolves the first record of work chunk k (the
// same chunk_start as the attribution launch that follows) with the per-lane
// search.  All chunks' lookups run in parallel here, so their dependent
// index loads overlap, instead of stalling one warp per chunk start inside
// the attribution (C5: ~10% of the attribution's stall samples were those
// searches).  The hint is only a candidate: the attribution re-checks that
// the object contains the record and is live at its timestamp (R5 makes such
// an object unique), else it searches as before.
#ifndef DRGPUM_HINT_MIN
#define DRGPUM_HINT_MIN (1ull << 28)   // launches with fewer records get no hints (C2, 1e8 records: the hint pass cost 2%)
#endif
__global__ void __launch_bounds__(256) chunk_hint_kernel(const __grid_constant__ AttrParams p, uint32_t n_warps) {
  __shared__ uint64_t s_l1[kL1MaxKeys];
  for (uint32_t i = threadIdx.x; i < p.n_l1; i += blockDim.x) s_l1[i] = p.l1[i];
  __syncthreads();
  ChunkHint* hints = const_cast<ChunkHint*>(p.hints);
  for (uint64_t k = uint64_t(blockIdx.x) * blockDim.x + threadIdx.x; k < p.hint_cap;
       k += uint64_t(gridDim.x) * blockDim.x) {
    const uint64_t i = chunk_start(k, p, n_warps);
    if (i >= p.n) break;                               // chunk starts grow with k
    const uint4 r = __ldg(p.recs + i);
    const uint64_t addr = (uint64_t(r.y) << 32) | r.x;
    const uint32_t ts = r.w & 0x7FFFFFFFu;
    uint32_t o = kNone, rank = kNone;
    DevObj d{};
    if (ts < p.n_api) rank = __ldg(p.acc_rank + ts);
    if (r.z != 0 && ts < p.n_api && addr <= ~0ull - r.z && rank != kNone) {
      o = find_object(p, s_l1, addr, ts);
      if (o != kNone) {
        d = p.objs[o];
        if (ts >= d.t_free) o = kNone;
      }
    }
    ChunkHint h;
    h.o = d; h.obj = o; h.pad[0] = r.w; h.pad[1] = rank; h.pad[2] = 0;   // pad: the first record's meta, its rank
    hints[k] = h;
  }
}

int attribute_occupancy() {
  int occ = 0;
  cudaFuncSetAttribute(attribute_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, int(kAttrSmem));
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, attribute_kernel, kAttrThreads, kAttrSmem);
  return occ < 1 ? 1 : occ;
}

int launch_attribute(const AttrParams& p, int num_sms, int occ, cudaStream_t s) {
  if (p.n == 0) return 0;
  // C_WORK and this call's queue count are zero here: zeroed by the reset,
  // then re-armed by the previous call's range_expand_kernel
  // enough stages per block to keep the ring busy, at most one wave
  uint64_t blocks = (p.n + 4ull * kConsumerWarps * kWarpRecords - 1) / (4ull * kConsumerWarps * kWarpRecords);
  const uint64_t full = uint64_t(num_sms) * occ;
  if (blocks > full) blocks = full;
  if (blocks < 1) blocks = 1;
  AttrParams q = p;
  q.chunk_shift = attribute_chunk_shift(p.n, blocks * kConsumerWarps, p.chunk_max_shift);
  chunk_bounds(q);
  int launches = 2;
  if (q.hint_cap && p.n >= DRGPUM_HINT_MIN) {
    const uint64_t kmax = p.n / 1024 + 2;              // chunks have >= 1024 records but the last
    q.hint_cap = uint32_t(kmax < q.hint_cap ? kmax : q.hint_cap);
    chunk_hint_kernel<<<(q.hint_cap + 255) / 256, 256, 0, s>>>(q, uint32_t(blocks * kConsumerWarps));
    ++launches;
  } else {
    q.hint_cap = 0;
  }
  attribute_kernel<<<(unsigned)blocks, kAttrThreads, kAttrSmem, s>>>(q);
  range_expand_kernel<<<num_sms * 4, 256, 0, s>>>(p.rq, p.ctr, p.rq_slot, p.rq_cap, p.orw);
  return launches;
}

}  // namespace drgpum

namespace drgpum {

// ------------------------------------------------------------------ NEXT-3
// Structured access (Def 3.10 l.200; §5.2 l.270): O matches if every GPU API
// that accesses O touches its own slice and no two slices overlap.  Exactly
// that, order-free: owner[e] holds (access rank + 1) of the first API that
// claimed element e (a CAS from 0); an API that finds another API's tag on an
// element marks O as overlapped.  Values only go 0 -> tag, so a stale plain
// read is either 0 (then the CAS decides) or already final.
__device__ __forceinline__ bool sa_claim(uint32_t* owner, uint32_t* overlap, uint64_t g, uint32_t tag,
                                         uint32_t obj) {
  uint32_t cur = owner[g];
  if (cur == 0) cur = atomicCAS(owner + g, 0u, tag);
  if (cur == 0 || cur == tag) return false;
  // one writer per object in the common case: the flag is read (L2) first so
  // that threads arriving after it is set do not serialise on its address
  if (!__ldcg(overlap + obj)) red_or(overlap + obj, 1u);
  return true;
}

constexpr uint32_t kSaInline = 64;          // elements claimed by the lane itself
constexpr uint64_t kSaChunk = 4096;         // queued work item (elements)

constexpr uint32_t kSaUnroll = 4;           // records per lane per round (independent chains)

// Queue a large element range (>= kSaInline elements) in kSaChunk pieces for
// structured_range_kernel; claims in place when the queue is full.
__device__ __noinline__ bool sa_enqueue(const SaParams& q, uint64_t g0, uint64_t g1, uint32_t tag, uint32_t obj) {
  const uint64_t nch = (g1 - g0) / kSaChunk + 1;
  const unsigned long long slot = atomicAdd(q.q_count, (unsigned long long)nch);
  bool dead = false;
  for (uint64_t k = 0; k < nch; ++k) {
    const uint64_t lo = g0 + k * kSaChunk, hi = min(g1, lo + kSaChunk - 1);
    if (slot + k < q.q_cap) {
      q.q[slot + k] = SaRange{lo, hi, obj, tag, {0, 0}};
    } else {
      for (uint64_t g = lo; g <= hi && !dead; ++g) dead = sa_claim(q.owner, q.overlap, g, tag, obj);
    }
  }
  return dead;
}

// Every warp owns a contiguous span of records and reads it 32 x kSaUnroll
// records per round (coalesced, streamed past L2), so a lane's consecutive
// records are 32 apart -- inside one burst, where its object and API caches
// hit.  The kSaUnroll records' owner reads are issued together before any
// CAS, so each lane keeps kSaUnroll independent load chains in flight.
__global__ void __launch_bounds__(256, 4) structured_kernel(const __grid_constant__ SaParams q) {
  const AttrParams& p = q.a;
  const int lane = threadIdx.x & 31;
  const uint64_t gw = (uint64_t(blockIdx.x) * blockDim.x + threadIdx.x) >> 5;
  const uint64_t nw = (uint64_t(gridDim.x) * blockDim.x) >> 5;
  constexpr uint64_t kRound = 32ull * kSaUnroll;
  const uint64_t per = ((p.n + nw - 1) / nw + kRound - 1) / kRound * kRound;
  const uint64_t w_lo = gw * per, w_hi = min(p.n, w_lo + per);
  // per-lane object cache (+ whether the cached object is already overlapped)
  uint64_t c_base = 0, c_size = 0, c_eb = 0;
  uint32_t c_ta = 0, c_tf = 0, c_obj = kNone, c_shift = 0;
  bool c_dead = false;
  uint32_t c_ts = ~0u, c_tag = 0;             // per-lane API cache: tag 0 = not in the pass
  for (uint64_t b = w_lo; b < w_hi; b += kRound) {
    // another lane or warp may have decided the cached object meanwhile: its
    // flag is re-read every round (in flight together with the records)
    const uint32_t ov_now = (c_obj != kNone && !c_dead) ? __ldcg(q.overlap + c_obj) : 0u;
    uint4 r[kSaUnroll];
#pragma unroll
    for (uint32_t k = 0; k < kSaUnroll; ++k) {
      const uint64_t i = b + k * 32 + uint64_t(lane);
      r[k] = i < w_hi ? __ldcs(p.recs + i) : make_uint4(0, 0, 0, 0);
    }
    if (ov_now) c_dead = true;
    uint64_t g[kSaUnroll];
    uint32_t cnt[kSaUnroll], tag[kSaUnroll], obj[kSaUnroll], cur[kSaUnroll];
#pragma unroll
    for (uint32_t k = 0; k < kSaUnroll; ++k) {
      cnt[k] = 0; g[k] = 0; tag[k] = 0; obj[k] = kNone;
      const uint64_t addr = (uint64_t(r[k].y) << 32) | r[k].x;
      const uint32_t size = r[k].z, ts = r[k].w & 0x7FFFFFFFu;
      if (size == 0 || ts >= p.n_api || addr > ~0ull - size) continue;
      if (ts != c_ts) {
        const uint32_t rank = __ldg(p.acc_rank + ts);
        c_ts = ts;
        c_tag = (rank == kNone || !__ldg(q.in_group + ts)) ? 0u : rank + 1;
      }
      if (c_tag == 0) continue;
      if (!(addr - c_base < c_size && ts > c_ta && ts < c_tf)) {
        const uint32_t o = find_object(p, p.l1, addr, ts);   // level-1 keys from global here
        if (o == kNone) continue;
        const DevObj d = p.objs[o];
        if (ts >= d.t_free) continue;
        c_base = d.base; c_size = d.end - d.base; c_ta = d.t_alloc; c_tf = d.t_free;
        c_obj = o; c_shift = d.shift; c_eb = __ldg(q.elem_base + o);
        c_dead = __ldcg(q.overlap + o) != 0;
      }
      if (c_dead) continue;
      const uint64_t off = addr - c_base;
      const uint64_t end = min(off + size, c_size);
      const uint64_t e0 = off >> c_shift, e1 = (end - 1) >> c_shift;
      if (e1 - e0 >= kSaInline) {
        c_dead = sa_enqueue(q, c_eb + e0, c_eb + e1, c_tag, c_obj);
        continue;
      }
      g[k] = c_eb + e0; cnt[k] = uint32_t(e1 - e0) + 1; tag[k] = c_tag; obj[k] = c_obj;
    }
#pragma unroll
    for (uint32_t k = 0; k < kSaUnroll; ++k) cur[k] = cnt[k] ? q.owner[g[k]] : 0u;
#pragma unroll
    for (uint32_t k = 0; k < kSaUnroll; ++k) {
      if (cnt[k] == 0) continue;
      bool dead = false;
      // first element: the owner value read above (0 -> the CAS decides)
      uint32_t c0 = cur[k];
      if (c0 == 0) c0 = atomicCAS(q.owner + g[k], 0u, tag[k]);
      if (c0 != 0 && c0 != tag[k]) {
        if (!__ldcg(q.overlap + obj[k])) red_or(q.overlap + obj[k], 1u);
        dead = true;
      }
      for (uint32_t e = 1; e < cnt[k] && !dead; ++e) dead = sa_claim(q.owner, q.overlap, g[k] + e, tag[k], obj[k]);
      if (dead && obj[k] == c_obj) c_dead = true;
    }
  }
}

__global__ void __launch_bounds__(256) structured_range_kernel(const __grid_constant__ SaParams q) {
  const unsigned long long raw = *q.q_count;
  const uint64_t cnt = raw < q.q_cap ? raw : q.q_cap;
  const int lane = threadIdx.x & 31;
  const uint64_t gwarp = (uint64_t(blockIdx.x) * blockDim.x + threadIdx.x) >> 5;
  const uint64_t nwarps = (uint64_t(gridDim.x) * blockDim.x) >> 5;
  for (uint64_t e = gwarp; e < cnt; e += nwarps) {
    const SaRange r = q.q[e];
    if (__ldcg(q.overlap + r.obj)) continue;
    for (uint64_t b = r.g_lo; b <= r.g_hi; b += 32) {     // warp-uniform trip count
      const uint64_t g = b + lane;
      const bool hit = g <= r.g_hi && sa_claim(q.owner, q.overlap, g, r.tag, r.obj);
      if (__any_sync(0xffffffffu, hit)) break;
    }
  }
}

int launch_structured(const SaParams& q, int num_sms, cudaStream_t s) {
  if (q.a.n == 0) return 0;
  cudaMemsetAsync(q.q_count, 0, sizeof(unsigned long long), s);
  // one round per warp at least; at most 4 blocks (32 warps) per SM
  uint64_t blocks = (q.a.n + 8 * 32 * kSaUnroll - 1) / (8 * 32 * kSaUnroll);
  if (blocks > uint64_t(num_sms) * 4) blocks = uint64_t(num_sms) * 4;
  structured_kernel<<<(unsigned)blocks, 256, 0, s>>>(q);
  structured_range_kernel<<<num_sms * 4, 256, 0, s>>>(q);
  return 2;
}

}  // namespace drgpum
