// B1 attribute_kernel + B2 range_expand_kernel (sm_100a).
//
// Per record (§5.1 l.238-240, §5.2 l.264-268):
//   A1  stream the 16-B record (ld.global.nc.L1::no_allocate, 128-bit),
//       reject invalid ones (size 0, ts >= n_api, ts of an ALLOC/FREE API --
//       footnote 2 l.178 --, addr+size overflow);
//   A2  find the object live at ts that contains addr: per-lane cache of the
//       last object (bursts are warp-coalesced), else a two-level search of
//       the static segment index (level-1 keys in shared memory, leaves in
//       L2) and a search of the segment's candidates by t_alloc (address
//       reuse, reading R5);
//   A3  clip to the object (R3), turn the byte range into element bits
//       (partial elements count, R2) and OR them into the object's bitmap:
//       lanes hitting the same u32 word are merged by a warp segmented scan
//       (or one REDUX when the whole warp hits one word) and a single RED.OR
//       per word run; ranges spanning > 2 words go to the range queue (A3b);
//   A4  fold ts into first (RED.MIN) / last (RED.MAX) and OR the (access API,
//       read|write) bit into the object's hit row -- both skipped when this
//       lane already knows the global value covers it (values are monotone);
//   A5  count records / attributed / unattributed / clipped / invalid.
#include "internal.cuh"

namespace drgpum {

#define FULL_MASK 0xFFFFFFFFu

__device__ __forceinline__ uint4 ld_stream(const uint4* p) {
  uint4 r;
  asm volatile("ld.global.nc.L1::no_allocate.L2::256B.v4.u32 {%0,%1,%2,%3}, [%4];"
               : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(p));
  return r;
}

__device__ __forceinline__ uint32_t bits_mask(uint32_t b0, uint32_t b1) {  // bits b0..b1 inclusive
  return (0xFFFFFFFFu >> (31 - b1)) & (0xFFFFFFFFu << b0);
}

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

// OR masks into words, one RED per run of lanes sharing a word.
__device__ __forceinline__ void warp_or_words(uint32_t* words, uint64_t key, uint32_t m, int lane) {
  const uint64_t k0 = __shfl_sync(FULL_MASK, key, 0);
  if (__all_sync(FULL_MASK, key == k0)) {
    const uint32_t v = __reduce_or_sync(FULL_MASK, m);
    if (lane == 0 && k0 != kNoKey && v) atomicOr(words + k0, v);
    return;
  }
  bool tail;
  const uint32_t v = seg_scan(key, m, lane, tail, OpOr());
  if (tail && key != kNoKey && v) atomicOr(words + key, v);
}

struct LaneCache {
  uint64_t base, end, bm_bit, hit_word;
  uint32_t t_alloc, t_free, r_lo, shift, obj;
  uint32_t ts, rank;          // last timestamp -> access-API rank
  uint32_t first_known;       // first[obj] <= first_known is known
  uint32_t last_known;        // last[obj]  >= last_known  is known
  uint64_t hw;                // hit word whose bits hbits are known set
  uint32_t hbits;
};

struct LaneCounts { uint32_t rec, attr, unattr, clip, inval, ovf; };

__device__ __forceinline__ uint32_t find_object(const AttrParams& p, const uint64_t* s_l1,
                                                uint64_t addr, uint32_t ts) {
  if (p.n_seg == 0 || addr < s_l1[0]) return kNone;
  // level 1 (shared memory): last key <= addr
  uint32_t lo = 0, hi = p.n_l1;
  while (hi - lo > 1) {
    const uint32_t mid = (lo + hi) >> 1;
    if (s_l1[mid] <= addr) lo = mid; else hi = mid;
  }
  // level 2 (global/L2): last segment start <= addr within the level-1 block
  uint32_t a = lo * p.l1_stride;
  uint32_t b = min(a + p.l1_stride, p.n_seg);
  while (b - a > 1) {
    const uint32_t mid = (a + b) >> 1;
    if (__ldg(p.seg_start + mid) <= addr) a = mid; else b = mid;
  }
  const uint32_t c0 = __ldg(p.seg_cand_off + a), c1 = __ldg(p.seg_cand_off + a + 1);
  if (c0 == c1) return kNone;
  // candidates sorted by t_alloc, lifetimes disjoint: the last one allocated
  // before ts is the only one that can be live at ts
  uint32_t l = c0, h = c1;
  const uint2* cand = reinterpret_cast<const uint2*>(p.cand);
  while (l < h) {
    const uint32_t mid = (l + h) >> 1;
    if (__ldg(&cand[mid].y) < ts) l = mid + 1; else h = mid;
  }
  if (l == c0) return kNone;
  return __ldg(&cand[l - 1].x);
}

__device__ __noinline__ void enqueue_range(const AttrParams& p, uint64_t gb0, uint64_t gb1, LaneCounts& k) {
  const uint64_t wlo = gb0 >> 5, whi = gb1 >> 5;
  const uint64_t nch = (whi - wlo) / kRangeChunkWords + 1;
  const unsigned long long slot = atomicAdd(&p.ctr[C_RQ_COUNT], (unsigned long long)nch);
  for (uint64_t c = 0; c < nch; ++c) {
    const uint64_t cw0 = wlo + c * kRangeChunkWords;
    const uint64_t bl = c == 0 ? gb0 : cw0 * 32;
    const uint64_t bh = min(gb1, (cw0 + kRangeChunkWords) * 32 - 1);
    if (slot + c < p.rq_cap) {
      p.rq[slot + c] = RangeEntry{bl, bh};
    } else {  // queue full: expand this chunk in place (slow but exact)
      k.ovf++;
      for (uint64_t w = bl >> 5; w <= (bh >> 5); ++w) {
        uint32_t m = 0xFFFFFFFFu;
        if (w == (bl >> 5)) m &= 0xFFFFFFFFu << (bl & 31);
        if (w == (bh >> 5)) m &= 0xFFFFFFFFu >> (31 - (bh & 31));
        atomicOr(p.orw + w, m);
      }
    }
  }
}

__device__ __forceinline__ void process(const AttrParams& p, const uint64_t* s_l1, uint4 r,
                                        bool present, int lane, LaneCache& c, LaneCounts& k) {
  const uint64_t addr = (uint64_t(r.y) << 32) | r.x;
  const uint32_t size = r.z;
  const uint32_t ts = r.w & 0x7FFFFFFFu;
  const uint32_t is_w = r.w >> 31;
  // ---- A1: validity
  bool ok = present && size != 0 && ts < p.n_api && addr <= ~0ull - size;
  if (ok && ts != c.ts) { c.rank = __ldg(p.acc_rank + ts); c.ts = ts; }
  ok = ok && c.rank != kNone;
  k.rec += present;
  k.inval += present && !ok;
  // ---- A2: object lookup
  bool att = false;
  if (ok) {
    att = addr >= c.base && addr < c.end && ts > c.t_alloc && ts < c.t_free;
    if (!att) {
      const uint32_t o = find_object(p, s_l1, addr, ts);
      if (o != kNone) {
        const uint4* q = reinterpret_cast<const uint4*>(p.objs + o);
        const uint4 a = __ldg(q), b = __ldg(q + 1), d = __ldg(q + 2);
        if (ts < d.y) {
          c.base = (uint64_t(a.y) << 32) | a.x;
          c.end = (uint64_t(a.w) << 32) | a.z;
          c.bm_bit = (uint64_t(b.y) << 32) | b.x;
          c.hit_word = (uint64_t(b.w) << 32) | b.z;
          c.t_alloc = d.x; c.t_free = d.y; c.r_lo = d.z; c.shift = d.w;
          c.obj = o;
          c.first_known = kNever; c.last_known = 0;
          c.hw = kNoKey; c.hbits = 0;
          att = true;
        }
      }
    }
    k.attr += att;
    k.unattr += !att;
  }
  // ---- A3: element bits
  uint64_t key0 = kNoKey, key1 = kNoKey;
  uint32_t m0 = 0, m1 = 0;
  if (att) {
    uint64_t end = addr + size;
    if (end > c.end) { end = c.end; k.clip++; }
    const uint64_t gb0 = c.bm_bit + ((addr - c.base) >> c.shift);
    const uint64_t gb1 = c.bm_bit + ((end - 1 - c.base) >> c.shift);
    const uint64_t w0 = gb0 >> 5, w1 = gb1 >> 5;
    if (w1 - w0 >= 2) {
      enqueue_range(p, gb0, gb1, k);
    } else if (w1 == w0) {
      key0 = w0; m0 = bits_mask(gb0 & 31, gb1 & 31);
    } else {
      key0 = w0; m0 = 0xFFFFFFFFu << (gb0 & 31);
      key1 = w1; m1 = 0xFFFFFFFFu >> (31 - (gb1 & 31));
    }
  }
  warp_or_words(p.orw, key0, m0, lane);
  if (__any_sync(FULL_MASK, key1 != kNoKey)) warp_or_words(p.orw, key1, m1, lane);
  // ---- A4: liveness fold
  const bool need_min = att && ts < c.first_known;
  if (__any_sync(FULL_MASK, need_min)) {
    bool tail;
    const uint64_t key = need_min ? c.obj : kNoKey;
    const uint32_t v = seg_scan(key, ts, lane, tail, OpMin());
    if (tail && need_min) atomicMin(p.first + c.obj, v);
    if (need_min) c.first_known = ts;
  }
  const bool need_max = att && ts > c.last_known;
  if (__any_sync(FULL_MASK, need_max)) {
    bool tail;
    const uint64_t key = need_max ? c.obj : kNoKey;
    const uint32_t v = seg_scan(key, ts, lane, tail, OpMax());
    if (tail && need_max) atomicMax(p.last + c.obj, v);
    if (need_max) c.last_known = ts;
  }
  // hit row: bit 2*(rank - r_lo) + is_write of the object's row
  uint64_t hkey = kNoKey;
  uint32_t hm = 0;
  if (att) {
    const uint32_t hb = 2 * (c.rank - c.r_lo) + is_w;
    const uint64_t hw = c.hit_word + (hb >> 5);
    const uint32_t bit = 1u << (hb & 31);
    if (!(hw == c.hw && (c.hbits & bit))) { hkey = hw; hm = bit; }
  }
  if (__any_sync(FULL_MASK, hkey != kNoKey)) {
    warp_or_words(p.orw, hkey, hm, lane);
    if (hkey != kNoKey) {
      if (hkey == c.hw) c.hbits |= hm; else { c.hw = hkey; c.hbits = hm; }
    }
  }
}

constexpr int kAttrThreads = 256;
constexpr int kAttrUnroll = 4;

__global__ void __launch_bounds__(kAttrThreads, 2) attribute_kernel(const AttrParams p) {
  __shared__ uint64_t s_l1[kL1MaxKeys];
  for (uint32_t i = threadIdx.x; i < p.n_l1; i += blockDim.x) s_l1[i] = p.l1[i];
  __syncthreads();
  const int lane = threadIdx.x & 31;
  const uint64_t gwarp = (uint64_t(blockIdx.x) * blockDim.x + threadIdx.x) >> 5;
  const uint64_t nwarps = (uint64_t(gridDim.x) * blockDim.x) >> 5;
  LaneCache c;
  c.base = 1; c.end = 0; c.bm_bit = 0; c.hit_word = 0;
  c.t_alloc = 0; c.t_free = 0; c.r_lo = 0; c.shift = 0; c.obj = kNone;
  c.ts = kNone; c.rank = kNone; c.first_known = kNever; c.last_known = 0;
  c.hw = kNoKey; c.hbits = 0;
  LaneCounts k = {0, 0, 0, 0, 0, 0};
  constexpr uint64_t per_iter = 32 * kAttrUnroll;
  for (uint64_t base = gwarp * per_iter; base < p.n; base += nwarps * per_iter) {
    uint4 r[kAttrUnroll];
#pragma unroll
    for (int u = 0; u < kAttrUnroll; ++u) {
      const uint64_t i = base + u * 32 + lane;
      r[u] = i < p.n ? ld_stream(p.recs + i) : make_uint4(0, 0, 0, 0);
    }
#pragma unroll
    for (int u = 0; u < kAttrUnroll; ++u)
      process(p, s_l1, r[u], base + u * 32 + lane < p.n, lane, c, k);
  }
  // A5: warp-reduce the counters, one atomic per warp and counter
  const uint32_t v[6] = {k.rec, k.attr, k.unattr, k.clip, k.inval, k.ovf};
  const int slot[6] = {C_RECORDS, C_ATTRIBUTED, C_UNATTRIBUTED, C_CLIPPED, C_INVALID, C_RQ_OVERFLOW};
#pragma unroll
  for (int i = 0; i < 6; ++i) {
    const uint32_t s = __reduce_add_sync(FULL_MASK, v[i]);
    if (lane == 0 && s) atomicAdd(&p.ctr[slot[i]], (unsigned long long)s);
  }
}

// B2: expand queued ranges: one warp per <= kRangeChunkWords-word entry;
// interior words get a plain all-ones store (idempotent with concurrent ORs),
// edge words a RED.OR.
__global__ void __launch_bounds__(256) range_expand_kernel(const RangeEntry* rq,
    const unsigned long long* ctr, uint32_t cap, uint32_t* orw) {
  const unsigned long long cnt_raw = ctr[C_RQ_COUNT];
  const uint64_t cnt = cnt_raw < cap ? cnt_raw : cap;
  const int lane = threadIdx.x & 31;
  const uint64_t gwarp = (uint64_t(blockIdx.x) * blockDim.x + threadIdx.x) >> 5;
  const uint64_t nwarps = (uint64_t(gridDim.x) * blockDim.x) >> 5;
  for (uint64_t e = gwarp; e < cnt; e += nwarps) {
    const RangeEntry r = rq[e];
    const uint64_t w0 = r.bit_lo >> 5, w1 = r.bit_hi >> 5;
    for (uint64_t w = w0 + lane; w <= w1; w += 32) {
      uint32_t m = 0xFFFFFFFFu;
      if (w == w0) m &= 0xFFFFFFFFu << (r.bit_lo & 31);
      if (w == w1) m &= 0xFFFFFFFFu >> (31 - (r.bit_hi & 31));
      if (m == 0xFFFFFFFFu) orw[w] = m; else atomicOr(orw + w, m);
    }
  }
}

int launch_attribute(const AttrParams& p, int num_sms, cudaStream_t s) {
  if (p.n == 0) return 0;
  cudaMemsetAsync(p.ctr + C_RQ_COUNT, 0, sizeof(unsigned long long), s);
  static int occ = 0;
  if (!occ) {
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, attribute_kernel, kAttrThreads, 0);
    if (occ < 1) occ = 1;
  }
  const uint64_t per_block = uint64_t(kAttrThreads / 32) * 32 * kAttrUnroll;
  uint64_t blocks = (p.n + per_block - 1) / per_block;
  const uint64_t full = uint64_t(num_sms) * occ;
  if (blocks > full) blocks = full;
  attribute_kernel<<<(unsigned)blocks, kAttrThreads, 0, s>>>(p);
  range_expand_kernel<<<num_sms * 4, 256, 0, s>>>(p.rq, p.ctr, p.rq_cap, p.orw);
  return 2;
}

}  // namespace drgpum
