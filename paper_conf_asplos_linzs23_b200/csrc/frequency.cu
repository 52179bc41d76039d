// NEXT-2 non-uniform access frequency (Def 3.9; §5.2
// l.271; fn 3 l.222 -- coefficient of variation).
//
// The paper keeps, per data object, a hashmap element -> access frequency,
// zeroes it when a GPU API that will access the object starts, counts every
// instrumented access of that API, and when the API finishes tests the
// variance of the frequencies.  Reading R22: the statistics run
// over the elements the API touched (the hashmap's cells); CV is the
// population coefficient of variation; NUAF at API A iff CV > X (20%),
// exactly: (n*S2 - S1^2) * 100^2 > X^2 * S1^2.
//
// B200 version: the paper's hashmap, one per API, all APIs at once.  The
// records of one API form a contiguous "segment" of the timestamp-sorted
// trace.  Every increment of an element's count returns the previous count
// c, so the (object, API) sums follow without a second pass: n += (c == 0),
// S1 += 1, S2 += 2c + 1.
//   1. freq_scan_kernel / freq_plan_kernel: run starts per timestamp, ordered
//      compaction into segments.
//   2. freq_count_kernel: records and element touches per (object, API)
//      slot (warp-aggregated).  A slot with ONE record needs no counting at
//      all -- each of its elements is touched exactly once (n = S1 = S2 =
//      its element count): every memcpy / memset.  The other slots' touches
//      size their segment's open-addressing table (capacity 2^k >= 2x
//      touches).
//   3. freq_table_plan_kernel: tables laid out by a prefix sum, cut into
//      batches of `budget` entries.
//   4. freq_apply_kernel (cooperative): per batch, zero the tables, insert
//      every record's elements (CAS on the key, add on the count), expand
//      wide records (> 64 elements) grid-wide; the segments of a batch are
//      independent, so they all run concurrently.  Segments that may continue
//      across an attribute call (the first and the last of a call) or whose
//      table would not fit keep their counts in per-element cells {API tag,
//      count} instead and run alone, in trace order, after the batches.
// Lanes accumulate locally while they stay in one slot, then in a small
// per-block shared-memory table, flushed to the global sums at the end.
#include <cooperative_groups.h>

#include "internal.cuh"

namespace cg = cooperative_groups;

namespace drgpum {

constexpr uint64_t kFreqInline = 64;         // wider records are expanded grid-wide
constexpr uint64_t kFreqChunk = 1024;        // elements per queue chunk (32 per lane)
constexpr int kU = 8;                        // elements in flight per lane
constexpr int kFreqThreads = 256;
constexpr uint64_t kNone64 = ~0ull;

// kU elements x0 + st*j at once (valid bits in v): first probes and the adds
// are issued back to back, so a lane waits for two round trips per kU elements
__device__ __forceinline__ void tbl_incr_many(FreqEntry* t, uint32_t logc, uint64_t x0, uint64_t st, uint32_t v,
                                              uint32_t (&prev)[kU]) {
  const uint32_t mask = (1u << logc) - 1;
  unsigned long long k[kU];
  uint32_t h[kU];
#pragma unroll
  for (int j = 0; j < kU; ++j)
    if (v >> j & 1) {
      const unsigned long long key = x0 + st * j + 1;
      h[j] = uint32_t((key * 0x9E3779B97F4A7C15ull) >> (64 - logc));
      k[j] = atomicCAS(&t[h[j]].key, 0ull, key);
    }
#pragma unroll
  for (int j = 0; j < kU; ++j)
    if (v >> j & 1) {
      const unsigned long long key = x0 + st * j + 1;
      while (k[j] != 0 && k[j] != key) {
        h[j] = (h[j] + 1) & mask;
        k[j] = atomicCAS(&t[h[j]].key, 0ull, key);
      }
    }
#pragma unroll
  for (int j = 0; j < kU; ++j)
    if (v >> j & 1) prev[j] = uint32_t(atomicAdd(&t[h[j]].cnt, 1ull));
}

// one key, `add` more touches; returns the count before them
__device__ __forceinline__ uint32_t tbl_add(FreqEntry* t, uint32_t logc, unsigned long long key, uint32_t add) {
  const uint32_t mask = (1u << logc) - 1;
  uint32_t h = uint32_t((key * 0x9E3779B97F4A7C15ull) >> (64 - logc));
  unsigned long long k = atomicCAS(&t[h].key, 0ull, key);
  while (k != 0 && k != key) {
    h = (h + 1) & mask;
    k = atomicCAS(&t[h].key, 0ull, key);
  }
  return uint32_t(atomicAdd(&t[h].cnt, (unsigned long long)add));
}

__device__ __forceinline__ void cell_incr_many(unsigned long long* cells, uint32_t tag, uint64_t x0, uint64_t st,
                                               uint32_t v, uint32_t (&prev)[kU]) {
#pragma unroll
  for (int j = 0; j < kU; ++j)
    if (v >> j & 1)
      asm volatile("red.relaxed.gpu.global.max.u64 [%0], %1;" ::"l"(cells + x0 + st * j),
                   "l"((unsigned long long)tag << 32) : "memory");
#pragma unroll
  for (int j = 0; j < kU; ++j)
    if (v >> j & 1) prev[j] = uint32_t(atomicAdd(cells + x0 + st * j, 1ull));
}

// Per-block (object, API) accumulators in shared memory.
constexpr int kBlkSlots = 16;
struct BlkAcc {
  unsigned long long slot[kBlkSlots], n[kBlkSlots], s1[kBlkSlots], s2[kBlkSlots];
};

__device__ __forceinline__ void blk_add(BlkAcc& b, unsigned long long* acc, uint64_t slot, uint64_t n,
                                        uint64_t s1, uint64_t s2) {
  const unsigned h = unsigned(slot) & (kBlkSlots - 1);
  for (int k = 0; k < kBlkSlots; ++k) {
    const unsigned j = (h + k) & (kBlkSlots - 1);
    unsigned long long cur = b.slot[j];
    if (cur == ~0ull) cur = atomicCAS(&b.slot[j], ~0ull, (unsigned long long)slot);
    if (cur == ~0ull || cur == slot) {
      atomicAdd(&b.n[j], (unsigned long long)n);
      atomicAdd(&b.s1[j], (unsigned long long)s1);
      atomicAdd(&b.s2[j], (unsigned long long)s2);
      return;
    }
  }
  atomicAdd(acc + 3 * slot, (unsigned long long)n);            // table full: straight to global
  atomicAdd(acc + 3 * slot + 1, (unsigned long long)s1);
  atomicAdd(acc + 3 * slot + 2, (unsigned long long)s2);
}

// flush the block table to the global accumulators and clear it (block-wide)
__device__ __forceinline__ void blk_flush(BlkAcc& b, unsigned long long* acc) {
  __syncthreads();
  if (threadIdx.x < kBlkSlots) {
    const unsigned j = threadIdx.x;
    const unsigned long long sl = b.slot[j];
    if (sl != ~0ull && b.s1[j]) {
      atomicAdd(acc + 3 * sl, b.n[j]);
      atomicAdd(acc + 3 * sl + 1, b.s1[j]);
      atomicAdd(acc + 3 * sl + 2, b.s2[j]);
    }
    b.slot[j] = ~0ull;
    b.n[j] = b.s1[j] = b.s2[j] = 0;
  }
  __syncthreads();
}

struct SlotAcc {
  uint64_t slot = ~0ull, n = 0, s1 = 0, s2 = 0;
  __device__ void flush(BlkAcc& b, unsigned long long* acc) {
    if (slot != ~0ull && s1) blk_add(b, acc, slot, n, s1, s2);
    n = s1 = s2 = 0;
  }
  __device__ void to(BlkAcc& b, unsigned long long* acc, uint64_t sl) {
    if (sl != slot) { flush(b, acc); slot = sl; }
  }
  __device__ void add(BlkAcc& b, unsigned long long* acc, uint64_t sl, uint32_t prev) {
    to(b, acc, sl);
    n += prev == 0;
    s1 += 1;
    s2 += 2ull * prev + 1;
  }
  __device__ void add_once(BlkAcc& b, unsigned long long* acc, uint64_t sl, uint64_t len) {
    to(b, acc, sl);            // len distinct elements, each touched once
    n += len;
    s1 += len;
    s2 += len;
  }
};

// object lookup (same index and rules as the attribution kernel)
__device__ __forceinline__ uint32_t freq_find(const AttrParams& p, const uint64_t* l1, uint64_t addr,
                                              uint32_t ts) {
  if (p.n_seg == 0 || addr < l1[0]) return kNone;
  uint32_t lo = 0, hi = p.n_l1;
  while (hi - lo > 1) { const uint32_t m = (lo + hi) >> 1; if (l1[m] <= addr) lo = m; else hi = m; }
  uint32_t a = lo * p.l1_stride, b = min(a + p.l1_stride, p.n_seg);
  while (b - a > 1) { const uint32_t m = (a + b) >> 1; if (p.seg_start[m] <= addr) a = m; else b = m; }
  const uint32_t c0 = p.seg_cand_off[a], c1 = p.seg_cand_off[a + 1];
  if (c0 == c1) return kNone;
  uint32_t l = c0, h = c1;
  while (l < h) { const uint32_t m = (l + h) >> 1; if (p.cand[m].t_alloc < ts) l = m + 1; else h = m; }
  return l == c0 ? kNone : p.cand[l - 1].obj;
}

__device__ __forceinline__ uint32_t ts_of(const AttrParams& p, uint64_t i) { return __ldcs(&p.recs[i].w) & 0x7FFFFFFFu; }

// A lane's cached object, and the element range / slot of one record.
struct LaneObj {
  uint64_t base = 0, size = 0, eb = 0, sb = 0;
  uint32_t ta = 0, tf = 0, rlo = 0, shift = 0;
};
struct Touch { uint64_t g0, g1, slot; };   // global elements [g0, g1]

// false if the record touches no live object (or is malformed)
__device__ __forceinline__ bool resolve(const FreqParams& q, const uint64_t* l1, LaneObj& c, uint64_t i,
                                        uint32_t t, uint32_t rank, Touch& out) {
  const AttrParams& p = q.a;
  const uint4 r = __ldcs(p.recs + i);                 // streamed: keep L2 for the tables
  const uint64_t addr = (uint64_t(r.y) << 32) | r.x;
  const uint32_t size = r.z;
  if (size == 0 || addr > ~0ull - size) return false;
  if (!(addr - c.base < c.size && t > c.ta && t < c.tf)) {
    const uint32_t o = freq_find(p, l1, addr, t);
    if (o == kNone) return false;
    const DevObj d = p.objs[o];
    if (t >= d.t_free) return false;
    c.base = d.base; c.size = d.end - d.base; c.ta = d.t_alloc; c.tf = d.t_free;
    c.rlo = d.r_lo; c.shift = d.shift;
    c.eb = q.elem_base[o]; c.sb = q.slot_base[o];
  }
  const uint64_t off = addr - c.base, end = min(off + size, c.size);
  out.g0 = c.eb + (off >> c.shift);
  out.g1 = c.eb + ((end - 1) >> c.shift);
  out.slot = c.sb + (rank - c.rlo);
  return true;
}

// every element of [g0, g1] (stride st, for lanes of a warp) touched once more
// in the table tb (lc) or, if tag != 0, in the element cells
struct Counter {
  FreqEntry* tb;
  unsigned long long* cells;
  uint32_t lc, tag;
  template <typename Acc>
  __device__ __forceinline__ void range(Acc& add, uint64_t g0, uint64_t g1, uint64_t st) const {
    for (uint64_t x0 = g0; x0 <= g1; x0 += st * kU) {
      uint32_t v = 0, prev[kU];
#pragma unroll
      for (int j = 0; j < kU; ++j)
        if (x0 + st * j <= g1) v |= 1u << j;
      if (tag) cell_incr_many(cells, tag, x0, st, v, prev);
      else tbl_incr_many(tb, lc, x0, st, v, prev);
#pragma unroll
      for (int j = 0; j < kU; ++j)
        if (v >> j & 1) add(prev[j]);
    }
  }
};

// 1. order check, run start per timestamp, start of the invalid-timestamp tail
__global__ void __launch_bounds__(256) freq_scan_kernel(const __grid_constant__ FreqParams q) {
  const AttrParams& p = q.a;
  const uint64_t tid = uint64_t(blockIdx.x) * blockDim.x + threadIdx.x;
  const uint64_t nth = uint64_t(gridDim.x) * blockDim.x;
  for (uint64_t i = tid; i < p.n; i += nth) {
    const uint32_t t = ts_of(p, i);
    const uint32_t tp = i ? ts_of(p, i - 1) : 0u;
    if (i && t < tp) atomicOr(q.state, 1u);
    if (i == 0 || t != tp) {
      if (t < p.n_api) q.run_start[t] = i;
      else atomicMin(reinterpret_cast<unsigned long long*>(q.run_start + p.n_api), (unsigned long long)i);
    }
  }
  if (tid == 0 && p.n && ts_of(p, 0) < q.state[1]) atomicOr(q.state, 1u);
}

// 1b. one block: ordered compaction of the run starts into segments
__global__ void __launch_bounds__(1024) freq_plan_kernel(const __grid_constant__ FreqParams q) {
  __shared__ uint32_t s_w[32];
  const AttrParams& p = q.a;
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, nw = blockDim.x >> 5;
  if (*reinterpret_cast<volatile uint32_t*>(q.state)) return;     // unsorted: ctl stays zero
  const uint32_t n_api = p.n_api;
  uint64_t base = 0;
  for (uint64_t c0 = 0; c0 < n_api; c0 += blockDim.x) {
    const uint64_t t = c0 + threadIdx.x;
    const uint64_t v = t < n_api ? q.run_start[t] : kNone64;
    const bool has = v != kNone64;
    const unsigned bal = __ballot_sync(0xffffffffu, has);
    if (lane == 0) s_w[warp] = __popc(bal);
    __syncthreads();
    uint32_t before = 0, round = 0;
    for (int w = 0; w < nw; ++w) { if (w < warp) before += s_w[w]; round += s_w[w]; }
    before += __popc(bal & ((1u << lane) - 1));
    if (has) {
      q.segs[base + before] = v;
      q.seg_of_ts[t] = uint32_t(base + before);
    }
    base += round;
    __syncthreads();
  }
  if (threadIdx.x == 0) {
    const uint64_t tail = q.run_start[n_api];
    const uint64_t end_valid = tail == kNone64 ? p.n : tail;
    q.segs[base] = end_valid;
    q.ctl->n_segs = base;
    q.ctl->end_valid = end_valid;
    q.state[1] = ts_of(p, p.n - 1);
  }
}

__device__ __forceinline__ bool is_boundary(uint64_t k, uint64_t n_segs) { return k == 0 || k + 1 == n_segs; }

// 2. records and element touches per slot (interior segments only)
__global__ void __launch_bounds__(256) freq_count_kernel(const __grid_constant__ FreqParams q) {
  __shared__ uint64_t s_l1[kL1MaxKeys];
  const AttrParams& p = q.a;
  for (uint32_t j = threadIdx.x; j < p.n_l1; j += blockDim.x) s_l1[j] = p.l1[j];
  __syncthreads();
  const uint64_t n_segs = q.ctl->n_segs, end = q.ctl->end_valid;
  // each warp walks one contiguous chunk (lane caches stay on one object)
  const uint64_t nwarps = (uint64_t(gridDim.x) * blockDim.x) >> 5;
  const uint64_t gw = (uint64_t(blockIdx.x) * blockDim.x + threadIdx.x) >> 5;
  const uint64_t chunk = ((end + nwarps - 1) / nwarps + 31) / 32 * 32;
  const uint64_t w_lo = min(end, gw * chunk), w_hi = min(end, w_lo + chunk);
  LaneObj c;
  for (uint64_t i = w_lo + (threadIdx.x & 31); i < w_lo + (w_hi - w_lo + 31) / 32 * 32; i += 32) {
    const uint64_t end_ = w_hi;
    unsigned long long slot = kNone64;
    uint64_t touches = 0;
    uint32_t k = 0;
    if (i < end_) {
      const uint32_t t = ts_of(p, i);
      const uint32_t rank = p.acc_rank[t];
      Touch tc;
      if (rank != kNone) {
        k = q.seg_of_ts[t];
        if (!is_boundary(k, n_segs) && resolve(q, s_l1, c, i, t, rank, tc)) {
          slot = tc.slot;
          touches = tc.g1 - tc.g0 + 1;
        }
      }
    }
    const unsigned grp = __match_any_sync(0xffffffffu, slot);
    const uint32_t lo16 = __reduce_add_sync(grp, uint32_t(touches & 0xFFFF));
    const uint32_t hi16 = __reduce_add_sync(grp, uint32_t(touches >> 16));
    if (slot != kNone64 && int(threadIdx.x & 31) == __ffs(grp) - 1) {
      const uint32_t old = atomicAdd(q.slot_recs + slot, uint32_t(__popc(grp)));
      atomicAdd(q.slot_touch + slot, (unsigned long long)hi16 * 65536ull + lo16);
      if (old == 0) {
        const unsigned long long at = atomicAdd(&q.ctl->n_list, 1ull);
        q.slot_list[at] = FreqSlotSeg{slot, k, 0};
      }
    }
  }
}

// 2b. touches that need a table, per segment (slots with more than one record)
__global__ void __launch_bounds__(256) freq_slotseg_kernel(const __grid_constant__ FreqParams q) {
  const uint64_t n = q.ctl->n_list;
  for (uint64_t j = uint64_t(blockIdx.x) * blockDim.x + threadIdx.x; j < n; j += uint64_t(gridDim.x) * blockDim.x) {
    const FreqSlotSeg e = q.slot_list[j];
    if (q.slot_recs[e.slot] > 1) atomicAdd(q.seg_touch + e.seg, q.slot_touch[e.slot]);
  }
}

// 3. one block: table capacities, prefix sum, batches, the ordered list of solo segments
__global__ void __launch_bounds__(1024) freq_table_plan_kernel(const __grid_constant__ FreqParams q) {
  __shared__ unsigned long long s_w[32];
  __shared__ uint32_t s_c[32];
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, nw = blockDim.x >> 5;
  const uint64_t n_segs = q.ctl->n_segs;
  const uint64_t B = q.budget;
  unsigned long long base = 0;
  uint64_t n_solo = 0;
  for (uint64_t c0 = 0; c0 < n_segs; c0 += blockDim.x) {
    const uint64_t k = c0 + threadIdx.x;
    bool solo = false;
    unsigned long long cap = 0;
    uint32_t logc = 0;
    if (k < n_segs) {
      solo = is_boundary(k, n_segs);
      const unsigned long long touch = q.seg_touch[k];
      if (!solo && touch) {
        const unsigned long long want = max(2ull * touch, 64ull);
        logc = 64 - __clzll(want - 1);
        cap = 1ull << logc;
        if (cap > B) { solo = true; cap = 0; logc = 0; }
      }
    }
    unsigned long long v = cap;                       // inclusive warp scan
    for (int d = 1; d < 32; d <<= 1) {
      const unsigned long long u = __shfl_up_sync(0xffffffffu, v, d);
      if (lane >= d) v += u;
    }
    if (lane == 31) s_w[warp] = v;
    const unsigned sb = __ballot_sync(0xffffffffu, solo);
    if (lane == 0) s_c[warp] = __popc(sb);
    __syncthreads();
    unsigned long long before = 0, round = 0;
    uint32_t sbefore = 0, sround = 0;
    for (int w = 0; w < nw; ++w) {
      if (w < warp) { before += s_w[w]; sbefore += s_c[w]; }
      round += s_w[w];
      sround += s_c[w];
    }
    if (k < n_segs) {
      if (solo) {
        q.solo[n_solo + sbefore + __popc(sb & ((1u << lane) - 1))] = uint32_t(k);
        q.seg_logcap[k] = kFreqSolo;
      } else {
        const unsigned long long my_base = base + before + v - cap;
        const uint64_t batch = my_base / B;
        const uint64_t off = my_base - batch * B;
        q.seg_logcap[k] = uint8_t(logc);
        q.seg_off[k] = off;
        if (batch < q.max_batches) {
          atomicMax(q.batch_extent + batch, (unsigned long long)(off + cap));
          atomicMin(q.batch_first + batch, uint32_t(k));
          atomicMax(&q.ctl->n_batches, (unsigned long long)(batch + 1));
        } else {
          atomicOr(q.state, 2u);                       // table plan overflow
        }
      }
    }
    __syncthreads();
    base += round;
    n_solo += sround;
  }
  if (threadIdx.x == 0) q.ctl->n_solo = n_solo;
}

struct ApplyShared {
  BlkAcc blk;
  uint64_t l1[kL1MaxKeys];
};

__global__ void __launch_bounds__(kFreqThreads, 2) freq_apply_kernel(const __grid_constant__ FreqParams q) {
  cg::grid_group g = cg::this_grid();
  __shared__ ApplyShared sh;
  const AttrParams& p = q.a;
  const uint64_t tid = uint64_t(blockIdx.x) * blockDim.x + threadIdx.x;
  const uint64_t nth = uint64_t(gridDim.x) * blockDim.x;
  const int lane = threadIdx.x & 31;
  const uint64_t gwarp = tid >> 5, nwarps = nth >> 5;
  if (threadIdx.x < kBlkSlots) {
    sh.blk.slot[threadIdx.x] = ~0ull;
    sh.blk.n[threadIdx.x] = sh.blk.s1[threadIdx.x] = sh.blk.s2[threadIdx.x] = 0;
  }
  for (uint32_t j = threadIdx.x; j < p.n_l1; j += blockDim.x) sh.l1[j] = p.l1[j];
  __syncthreads();
  if (*reinterpret_cast<volatile uint32_t*>(q.state)) return;     // uniform across the grid
  const uint64_t n_segs = q.ctl->n_segs, n_batches = q.ctl->n_batches, n_solo = q.ctl->n_solo;
  LaneObj c;
  SlotAcc sa;
  uint64_t q_done = 0;
  // a record wider than kFreqInline elements: queued in 4096-element chunks
  // (tag != 0: cells of a solo segment, else the table of segment `seg`)
  auto counter = [&](uint32_t tag, uint32_t seg) {
    Counter ct;
    ct.cells = q.cells;
    ct.tag = tag;
    ct.lc = tag ? 0u : q.seg_logcap[seg];
    ct.tb = tag ? q.table : q.table + q.seg_off[seg];
    return ct;
  };
  // a record wider than kFreqInline elements: queued in kFreqChunk-element
  // chunks (tag != 0: cells of a solo segment, else the table of segment `seg`)
  auto queue_range = [&](const Touch& tc, uint32_t tag, uint32_t seg) {
    const uint64_t nch = (tc.g1 - tc.g0) / kFreqChunk + 1;
    const unsigned long long s0 = atomicAdd(&q.ctl->q_count, (unsigned long long)nch);
    for (uint64_t j = 0; j < nch; ++j) {
      const uint64_t l0 = tc.g0 + j * kFreqChunk, h0 = min(tc.g1, l0 + kFreqChunk - 1);
      if (s0 + j < q.q_cap) {
        q.q[s0 + j] = FreqChunk{l0, h0, tc.slot, tag, seg};
      } else {
        const uint64_t sl = tc.slot;
        auto add = [&](uint32_t pv) { sa.add(sh.blk, q.acc, sl, pv); };
        counter(tag, seg).range(add, l0, h0, 1);
      }
    }
  };
  // this phase's queued chunks, grid-wide, one warp per chunk
  auto drain = [&]() {
    g.sync();
    const unsigned long long raw = *reinterpret_cast<volatile unsigned long long*>(&q.ctl->q_count);
    const uint64_t qc = raw < q.q_cap ? raw : q.q_cap;
    for (uint64_t e = q_done + gwarp; e < qc; e += nwarps) {
      const FreqChunk fr = q.q[e];
      const uint64_t sl = fr.slot;
      auto add = [&](uint32_t pv) { sa.add(sh.blk, q.acc, sl, pv); };
      if (fr.g_lo + lane <= fr.g_hi) counter(fr.tag, fr.seg).range(add, fr.g_lo + lane, fr.g_hi, 32);
    }
    q_done = raw;
    g.sync();
  };

  // 4a. batches of interior segments with per-API tables, all segments of a batch at once
  for (uint64_t b = 0; b < n_batches; ++b) {
    const uint32_t f = q.batch_first[b];
    if (f == kNone) continue;
    uint64_t nxt = n_segs;
    for (uint64_t b2 = b + 1; b2 < n_batches; ++b2)
      if (q.batch_first[b2] != kNone) { nxt = q.batch_first[b2]; break; }
    const uint64_t rec_lo = q.segs[f], rec_hi = q.segs[nxt];
    const uint64_t ext = q.batch_extent[b];
    uint4* tz = reinterpret_cast<uint4*>(q.table);
    for (uint64_t e = tid; e < ext; e += nth) tz[e] = make_uint4(0, 0, 0, 0);
    g.sync();
    uint32_t c_t = kNever, c_rank = kNone, c_k = 0;
    uint8_t c_lc = 0;
    FreqEntry* c_tb = q.table;
    const uint64_t chunk = ((rec_hi - rec_lo + nwarps - 1) / nwarps + 31) / 32 * 32;
    const uint64_t w_lo = min(rec_hi, rec_lo + gwarp * chunk), w_hi = min(rec_hi, w_lo + chunk);
    for (uint64_t i0 = w_lo; i0 < w_hi; i0 += 32) {         // contiguous per warp, warp-uniform
      const uint64_t i = i0 + lane;
      Touch tc;
      bool tbl = false;
      if (i < w_hi) {
        const uint32_t t = ts_of(p, i);
        if (t != c_t) {
          c_t = t;
          c_rank = p.acc_rank[t];
          c_k = q.seg_of_ts[t];
          c_lc = q.seg_logcap[c_k];
          c_tb = q.table + q.seg_off[c_k];
        }
        if (c_rank != kNone && c_lc != kFreqSolo && resolve(q, sh.l1, c, i, t, c_rank, tc)) {
          if (q.slot_recs[tc.slot] == 1)                   // the slot's only record
            sa.add_once(sh.blk, q.acc, tc.slot, tc.g1 - tc.g0 + 1);
          else if (tc.g1 - tc.g0 < kFreqInline)
            tbl = true;
          else
            queue_range(tc, 0u, c_k);
        }
      }
      // table touches, element by element, lanes hitting the same (table,
      // element) merged into one add (hot elements of random bursts)
      const uint64_t len = tbl ? tc.g1 - tc.g0 + 1 : 0;
      const uint32_t max_len = __reduce_max_sync(0xffffffffu, uint32_t(len));
      for (uint32_t j = 0; j < max_len; ++j) {
        const unsigned long long key = j < len ? tc.g0 + j + 1 : 0ull;
        const unsigned grp = __match_any_sync(0xffffffffu, key) & __match_any_sync(0xffffffffu, c_k);
        const int leader = __ffs(grp) - 1;
        uint32_t base = 0;
        if (key && lane == leader) base = tbl_add(c_tb, c_lc, key, __popc(grp));
        base = __shfl_sync(0xffffffffu, base, leader);
        if (key) sa.add(sh.blk, q.acc, tc.slot, base + __popc(grp & ((1u << lane) - 1)));
      }
    }
    drain();
  }
  // 4b. solo segments (call boundaries, oversized tables), one at a time, in trace order
  for (uint64_t s = 0; s < n_solo; ++s) {
    const uint32_t k = q.solo[s];
    const uint64_t rec_lo = q.segs[k], rec_hi = q.segs[k + 1];
    const uint32_t t = ts_of(p, rec_lo);
    const uint32_t rank = p.acc_rank[t];
    if (rank == kNone) continue;
    const uint32_t tag = rank + 1;
    const uint64_t chunk = ((rec_hi - rec_lo + nwarps - 1) / nwarps + 31) / 32 * 32;
    const uint64_t w_lo = min(rec_hi, rec_lo + gwarp * chunk), w_hi = min(rec_hi, w_lo + chunk);
    for (uint64_t i = w_lo + lane; i < w_hi; i += 32) {
      Touch tc;
      if (!resolve(q, sh.l1, c, i, t, rank, tc)) continue;
      if (tc.g1 - tc.g0 < kFreqInline) {
        const uint64_t sl = tc.slot;
        auto add = [&](uint32_t pv) { sa.add(sh.blk, q.acc, sl, pv); };
        counter(tag, k).range(add, tc.g0, tc.g1, 1);
      } else {
        queue_range(tc, tag, k);
      }
    }
    drain();
  }
  sa.flush(sh.blk, q.acc);
  blk_flush(sh.blk, q.acc);
}

// per object: the APIs at which it matches NUAF, and the first of them
__global__ void __launch_bounds__(256) frequency_reduce_kernel(const FreqReduceParams q) {
  for (uint64_t o = uint64_t(blockIdx.x) * blockDim.x + threadIdx.x; o < q.n_obj;
       o += uint64_t(gridDim.x) * blockDim.x) {
    const uint64_t sb = q.slot_base[o];
    const uint32_t nh = q.n_hit[o], r_lo = q.objs[o].r_lo;
    uint32_t cnt = 0, first = kNever;
    using u128 = unsigned __int128;
    for (uint32_t k = 0; k < nh; ++k) {
      const unsigned long long* a = q.acc + 3 * (sb + k);
      const u128 n = a[0], s1 = a[1], s2 = a[2];
      if (!s1) continue;
      // CV^2 = (n*S2 - S1^2)/S1^2 > (pct/100)^2
      if ((n * s2 - s1 * s1) * 10000u > u128(q.pct) * q.pct * s1 * s1) {
        ++cnt;
        if (first == kNever) first = q.acc_ts[r_lo + k];
      }
    }
    q.out_count[o] = cnt;
    q.out_first[o] = first;
  }
}

int frequency_occupancy() {
  int occ = 0;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, freq_apply_kernel, kFreqThreads, 0);
  if (occ < 1) occ = 1;
  return occ > 2 ? 2 : occ;
}

int launch_frequency(const FreqParams& q, uint64_t n_slots, int num_sms, int occ, cudaStream_t s) {
  if (q.a.n == 0) return 0;
  const uint64_t n_api = q.a.n_api;
  cudaMemsetAsync(q.ctl, 0, sizeof(FreqCtl), s);
  cudaMemsetAsync(q.run_start, 0xFF, 8 * (n_api + 1), s);
  cudaMemsetAsync(q.seg_touch, 0, 8 * (n_api + 1), s);
  cudaMemsetAsync(q.batch_first, 0xFF, 4 * (uint64_t(q.max_batches) + 1), s);
  cudaMemsetAsync(q.batch_extent, 0, 8 * uint64_t(q.max_batches), s);
  if (n_slots) {
    cudaMemsetAsync(q.slot_recs, 0, 4 * n_slots, s);
    cudaMemsetAsync(q.slot_touch, 0, 8 * n_slots, s);
  }
  uint64_t b = (q.a.n + 255) / 256;
  if (b > uint64_t(num_sms) * 8) b = uint64_t(num_sms) * 8;
  freq_scan_kernel<<<(unsigned)b, 256, 0, s>>>(q);
  freq_plan_kernel<<<1, 1024, 0, s>>>(q);
  freq_count_kernel<<<(unsigned)b, 256, 0, s>>>(q);
  freq_slotseg_kernel<<<num_sms, 256, 0, s>>>(q);
  freq_table_plan_kernel<<<1, 1024, 0, s>>>(q);
  void* args[] = {const_cast<FreqParams*>(&q)};
  cudaLaunchCooperativeKernel((void*)freq_apply_kernel, dim3(num_sms * occ), dim3(kFreqThreads), args, 0, s);
  return 6;
}

int launch_frequency_reduce(const FreqReduceParams& q, int num_sms, cudaStream_t s) {
  if (q.n_obj == 0) return 0;
  uint64_t b = (q.n_obj + 255) / 256;
  if (b > uint64_t(num_sms) * 8) b = uint64_t(num_sms) * 8;
  frequency_reduce_kernel<<<(unsigned)b, 256, 0, s>>>(q);
  return 1;
}

}  // namespace drgpum
