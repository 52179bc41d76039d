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
// B200 version.  The records of one API form a contiguous "segment" of the
// timestamp-sorted trace.  Each element owns a 64-bit cell {API tag, count};
// a red.max to {tag, 0} followed by an atom.add returns the element's previous
// count c in this API, so the (object, API) sums follow without a second pass:
// n += (c == 0), S1 += 1, S2 += 2c + 1.  The max is only correct if, for every
// object, the touches of earlier APIs are done before a later API touches it;
// nothing else needs ordering.  So segments run CONCURRENTLY:
//   * freq_scan_kernel / freq_plan_kernel find the segments (run starts per
//     timestamp, ordered compaction) and, per segment, how many 2048-record
//     work tiles overlap it (seg_left);
//   * freq_main_kernel (persistent blocks) pulls tiles in trace order.  Before
//     a lane touches object O for segment k it looks up, in O's hit row (which
//     the attribution kernel has just built), the previous API that accessed
//     O; if that API is a segment of this call whose seg_left is not yet zero,
//     the record is deferred and retried (the block drains the wide-record
//     queue while it waits, so waiting never blocks progress).  Each finished
//     tile part / queue chunk decrements its segment's seg_left.
//   * Wide records (> 64 elements) become 4096-element queue chunks that any
//     block expands (8 independent elements in flight per lane); a record that
//     is the only one of its segment on its object (a memcpy / memset) needs
//     no cells at all: each of its elements is touched once.
// Lanes accumulate locally while they stay in one (object, API) slot, then in
// a small per-block shared-memory table flushed once per tile part.
#include "internal.cuh"

namespace drgpum {

constexpr uint64_t kFreqInline = 64;         // wider records go to the chunk queue
constexpr uint64_t kFreqChunk = 4096;        // elements per queue chunk
constexpr uint32_t kFreqTile = 512;          // records per work tile (short chain steps)
constexpr int kFreqThreads = 256;

__device__ __forceinline__ void freq_claim(unsigned long long* cell, uint32_t tag) {
  asm volatile("red.relaxed.gpu.global.max.u64 [%0], %1;" ::"l"(cell), "l"((unsigned long long)tag << 32)
               : "memory");
}
__device__ __forceinline__ uint32_t freq_incr(unsigned long long* cell, uint32_t tag) {
  freq_claim(cell, tag);
  return uint32_t(atomicAdd(cell, 1ull));
}
__device__ __forceinline__ uint32_t ld_acquire_u32(const uint32_t* p) {
  uint32_t v;
  asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_release_u32(uint32_t* p, uint32_t v) {
  asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ unsigned long long ld_volatile_u64(const unsigned long long* p) {
  return *reinterpret_cast<const volatile unsigned long long*>(p);
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
  __device__ void add(BlkAcc& b, unsigned long long* acc, uint64_t sl, uint32_t prev) {
    if (sl != slot) { flush(b, acc); slot = sl; }
    n += prev == 0;
    s1 += 1;
    s2 += 2ull * prev + 1;
  }
};

// object lookup (same index and rules as the attribution kernel); l1 = the
// level-1 keys, staged in shared memory by the main kernel
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

__device__ __forceinline__ uint32_t ts_of(const AttrParams& p, uint64_t i) { return p.recs[i].w & 0x7FFFFFFFu; }

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

// 2. one block: ordered compaction of the run starts into segments, the tiles
//    overlapping each segment, the control block for the main kernel
__global__ void __launch_bounds__(1024) freq_plan_kernel(const __grid_constant__ FreqParams q) {
  __shared__ uint32_t s_w[32];
  const AttrParams& p = q.a;
  FreqCtl* ctl = q.ctl;
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, nw = blockDim.x >> 5;
  if (*reinterpret_cast<volatile uint32_t*>(q.state)) return;     // unsorted: ctl stays zero
  constexpr uint64_t kNone64 = ~0ull;
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
  const uint64_t n_segs = base;
  const uint64_t tail = q.run_start[n_api];
  const uint64_t end_valid = tail == kNone64 ? p.n : tail;
  if (threadIdx.x == 0) {
    q.segs[n_segs] = end_valid;
    uint32_t rank_first = kNone;
    for (uint64_t k = 0; k < n_segs && rank_first == kNone; ++k) rank_first = p.acc_rank[ts_of(p, q.segs[k])];
    ctl->n_segs = n_segs;
    ctl->n_tiles = (end_valid + kFreqTile - 1) / kFreqTile;
    ctl->end_valid = end_valid;
    ctl->rank_first = rank_first;
    ctl->gen = q.state[2] + 1u;
    q.state[2] = uint32_t(ctl->gen);
    q.state[1] = ts_of(p, p.n - 1);
  }
  __syncthreads();
  for (uint64_t k = threadIdx.x; k < n_segs; k += blockDim.x) {
    const uint64_t lo = q.segs[k], hi = q.segs[k + 1];
    q.seg_left[k] = uint32_t((hi - 1) / kFreqTile - lo / kFreqTile + 1);
  }
}

// Per-lane state of the main kernel: cached object and the last (segment,
// object) whose predecessor was found complete.
struct LaneObj {
  uint64_t base = 0, size = 0, eb = 0, sb = 0, hit = 0;
  uint32_t ta = 0, tf = 0, rlo = 0, shift = 0, obj = kNone;
  uint64_t ready_seg = ~0ull;
  uint32_t ready_obj = kNone;
};

// Has the previous API that accessed object c (before access rank `rank`)
// finished in this call?  Earlier calls are complete by stream order.
__device__ bool pred_done(const FreqParams& q, const LaneObj& c, uint32_t rank) {
  const uint32_t rank_first = uint32_t(q.ctl->rank_first);
  if (rank <= rank_first || rank <= c.rlo) return true;
  const uint32_t* row = q.a.orw + c.hit;
  const uint32_t lo_slot = rank_first > c.rlo ? rank_first - c.rlo : 0;   // slots of this call
  const uint64_t b = 2ull * (rank - c.rlo);                                 // bits [0, b) = earlier APIs
  int64_t w = int64_t(b >> 5);
  uint32_t word = (b & 31) ? (row[w] & ((1u << (b & 31)) - 1)) : 0u;
  const int64_t w_stop = int64_t((2ull * lo_slot) >> 5);
  while (!word && w > w_stop) word = row[--w];
  if (!word) return true;
  const uint32_t slot = uint32_t((uint64_t(w) * 32 + 31 - __clz(word)) >> 1);
  if (slot < lo_slot) return true;
  const uint32_t j_ts = q.acc_ts[c.rlo + slot];
  return ld_acquire_u32(q.seg_left + q.seg_of_ts[j_ts]) == 0;
}

struct MainShared {
  BlkAcc blk;
  uint64_t l1[kL1MaxKeys];
  uint32_t def[2][kFreqTile];       // deferred record indices (offsets into the tile part)
  uint32_t ndef[2];
  uint32_t amask;                   // records handled in closed form (small segments)
  int kind;                         // 0 exit / nothing, 1 tile, 2 chunk
  unsigned long long work;
  FreqChunk chunk;
};

// expand a queue chunk with the whole block
__device__ void run_chunk(const FreqParams& q, MainShared& sh, uint64_t h, uint32_t gen) {
  if (threadIdx.x == 0) {
    while (ld_acquire_u32(&q.q[h].ready) != gen) __nanosleep(64);
    sh.chunk = q.q[h];
  }
  __syncthreads();
  const FreqChunk fr = sh.chunk;
  SlotAcc sa;
  constexpr int kU = 8;
  constexpr uint64_t kT = kFreqThreads;
  for (uint64_t x0 = fr.g_lo + threadIdx.x; x0 <= fr.g_hi; x0 += kT * kU) {
    uint32_t c[kU];
#pragma unroll
    for (int j = 0; j < kU; ++j)
      if (x0 + kT * j <= fr.g_hi) freq_claim(q.cells + x0 + kT * j, fr.tag);
#pragma unroll
    for (int j = 0; j < kU; ++j)
      if (x0 + kT * j <= fr.g_hi) c[j] = uint32_t(atomicAdd(q.cells + x0 + kT * j, 1ull));
#pragma unroll
    for (int j = 0; j < kU; ++j)
      if (x0 + kT * j <= fr.g_hi) sa.add(sh.blk, q.acc, fr.slot, c[j]);
  }
  sa.flush(sh.blk, q.acc);
  blk_flush(sh.blk, q.acc);
  __threadfence();
  __syncthreads();
  if (threadIdx.x == 0) atomicSub(q.seg_left + fr.seg, 1u);
}

// thread 0: try to claim a queued chunk; true if one was claimed
__device__ bool claim_chunk(const FreqParams& q, unsigned long long* out) {
  FreqCtl* ctl = q.ctl;
  for (;;) {
    const unsigned long long h = ld_volatile_u64(&ctl->q_head), t = ld_volatile_u64(&ctl->q_tail);
    if (h >= t || h >= q.q_cap) return false;
    if (atomicCAS(&ctl->q_head, h, h + 1) == h) { *out = h; return true; }
  }
}

// One record of segment k (API `rank`, timestamp t).  Returns false if it
// must be deferred (its object's previous API is still running).
__device__ bool do_record(const FreqParams& q, MainShared& sh, LaneObj& c, SlotAcc& sa, uint64_t i,
                          uint64_t k, uint32_t t, uint32_t rank, uint32_t gen) {
  const AttrParams& p = q.a;
  const uint4 r = p.recs[i];
  const uint64_t addr = (uint64_t(r.y) << 32) | r.x;
  const uint32_t size = r.z;
  if (size == 0 || addr > ~0ull - size) return true;
  if (!(addr - c.base < c.size && t > c.ta && t < c.tf)) {
    const uint32_t o = freq_find(p, sh.l1, addr, t);
    if (o == kNone) return true;
    const DevObj d = p.objs[o];
    if (t >= d.t_free) return true;
    c.base = d.base; c.size = d.end - d.base; c.ta = d.t_alloc; c.tf = d.t_free;
    c.rlo = d.r_lo; c.shift = d.shift; c.hit = d.hit_word; c.obj = o;
    c.eb = q.elem_base[o]; c.sb = q.slot_base[o];
  }
  if (c.ready_seg != k || c.ready_obj != c.obj) {
    if (!pred_done(q, c, rank)) return false;
    c.ready_seg = k;
    c.ready_obj = c.obj;
  }
  const uint64_t off = addr - c.base, end = min(off + size, c.size);
  const uint64_t e0 = off >> c.shift, e1 = (end - 1) >> c.shift;
  const uint64_t slot = c.sb + (rank - c.rlo);
  const uint32_t tag = rank + 1;
  unsigned long long* cell = q.cells + c.eb;
  if (e1 - e0 < kFreqInline) {
    for (uint64_t e = e0; e <= e1; e += 4) {           // up to 4 elements in flight
      uint32_t cnt[4];
#pragma unroll
      for (int j = 0; j < 4; ++j) if (e + j <= e1) freq_claim(cell + e + j, tag);
#pragma unroll
      for (int j = 0; j < 4; ++j) if (e + j <= e1) cnt[j] = uint32_t(atomicAdd(cell + e + j, 1ull));
#pragma unroll
      for (int j = 0; j < 4; ++j) if (e + j <= e1) sa.add(sh.blk, q.acc, slot, cnt[j]);
    }
    return true;
  }
  const uint64_t nch = (e1 - e0) / kFreqChunk + 1;
  const unsigned long long s0 = atomicAdd(&q.ctl->q_tail, (unsigned long long)nch);
  const uint64_t queued = s0 < q.q_cap ? min(nch, uint64_t(q.q_cap - s0)) : 0;
  if (queued) atomicAdd(q.seg_left + k, uint32_t(queued));   // before any chunk can finish
  for (uint64_t j = 0; j < nch; ++j) {
    const uint64_t l0 = e0 + j * kFreqChunk, h0 = min(e1, l0 + kFreqChunk - 1);
    if (j < queued) {
      FreqChunk& it = q.q[s0 + j];
      it.g_lo = c.eb + l0; it.g_hi = c.eb + h0; it.slot = slot; it.tag = tag; it.seg = uint32_t(k);
      st_release_u32(&it.ready, gen);
    } else {
      for (uint64_t e = l0; e <= h0; ++e) sa.add(sh.blk, q.acc, slot, freq_incr(cell + e, tag));
    }
  }
  return true;
}

__global__ void __launch_bounds__(kFreqThreads, 2) freq_main_kernel(const __grid_constant__ FreqParams q) {
  __shared__ MainShared sh;
  const AttrParams& p = q.a;
  FreqCtl* ctl = q.ctl;
  const uint64_t n_tiles = ctl->n_tiles, n_segs = ctl->n_segs, end_valid = ctl->end_valid;
  const uint32_t gen = uint32_t(ctl->gen);
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  if (threadIdx.x < kBlkSlots) {
    sh.blk.slot[threadIdx.x] = ~0ull;
    sh.blk.n[threadIdx.x] = sh.blk.s1[threadIdx.x] = sh.blk.s2[threadIdx.x] = 0;
  }
  for (uint32_t j = threadIdx.x; j < p.n_l1; j += kFreqThreads) sh.l1[j] = p.l1[j];
  LaneObj c;
  for (;;) {
    if (threadIdx.x == 0) {
      int kind = 0;
      unsigned long long work = 0;
      for (;;) {
        if (claim_chunk(q, &work)) { kind = 2; break; }
        if (ld_volatile_u64(&ctl->tile_next) < n_tiles) {
          work = atomicAdd(&ctl->tile_next, 1ull);
          if (work < n_tiles) { kind = 1; break; }
        }
        if (ld_volatile_u64(&ctl->tiles_done) == n_tiles) {
          __threadfence();
          const unsigned long long h = ld_volatile_u64(&ctl->q_head), t = ld_volatile_u64(&ctl->q_tail);
          if (h >= t || h >= q.q_cap) break;                  // kind 0: all work handed out
        }
        __nanosleep(256);
      }
      sh.kind = kind;
      sh.work = work;
    }
    __syncthreads();
    const int kind = sh.kind;
    const unsigned long long work = sh.work;
    __syncthreads();
    if (kind == 0) break;
    if (kind == 2) { run_chunk(q, sh, work, gen); continue; }

    // a tile: records [w_lo, w_hi), in segment parts
    const uint64_t w_lo = work * kFreqTile, w_hi = min(w_lo + kFreqTile, end_valid);
    uint64_t k = q.seg_of_ts[ts_of(p, w_lo)];
    for (uint64_t lo = w_lo; lo < w_hi; ++k) {
      const uint64_t seg_lo = q.segs[k], seg_hi = q.segs[k + 1];
      const uint64_t hi = min(seg_hi, w_hi);
      const uint32_t t = ts_of(p, lo);
      const uint32_t rank = p.acc_rank[t];
      if (rank != kNone) {
        // small segment wholly inside this tile (and not continued across a
        // call boundary): a record that is its segment's only one on its
        // object touches each of its elements exactly once
        if (threadIdx.x == 0) { sh.amask = 0; sh.ndef[0] = 0; }
        __syncthreads();
        if (warp == 0 && seg_lo >= w_lo && seg_hi <= w_hi && seg_hi - seg_lo <= 32 && k > 0 &&
            k + 1 < n_segs) {
          const uint64_t i = lo + lane;
          uint32_t o = kNone;
          uint64_t len = 0;
          if (i < hi) {
            const uint4 r = p.recs[i];
            const uint64_t addr = (uint64_t(r.y) << 32) | r.x;
            if (r.z != 0 && addr <= ~0ull - r.z) {
              o = freq_find(p, sh.l1, addr, t);
              if (o != kNone) {
                const DevObj d = p.objs[o];
                if (t >= d.t_free) {
                  o = kNone;
                } else {
                  const uint64_t off = addr - d.base, end = min(off + r.z, d.end - d.base);
                  len = ((end - 1) >> d.shift) - (off >> d.shift) + 1;
                }
              }
            }
          }
          const unsigned same = __match_any_sync(0xffffffffu, o);
          bool alone = o != kNone && __popc(same) == 1;
          if (alone) {
            // still a link of O's chain: this segment may only complete after
            // O's previous API did, so the closed form needs that too
            LaneObj tmp;
            const DevObj d = p.objs[o];
            tmp.rlo = d.r_lo;
            tmp.hit = d.hit_word;
            alone = pred_done(q, tmp, rank);
          }
          if (alone) {
            const uint64_t slot = q.slot_base[o] + (rank - p.objs[o].r_lo);
            blk_add(sh.blk, q.acc, slot, len, len, len);
          }
          const unsigned m = __ballot_sync(0xffffffffu, alone || (i < hi && o == kNone));
          if (lane == 0) sh.amask = m;
        }
        __syncthreads();
        const uint32_t amask = sh.amask;
        SlotAcc sa;
        for (uint64_t i = lo + threadIdx.x; i < hi; i += kFreqThreads) {
          if (i - lo < 32 && ((amask >> (i - lo)) & 1u)) continue;
          if (!do_record(q, sh, c, sa, i, k, t, rank, gen))
            sh.def[0][atomicAdd(&sh.ndef[0], 1u)] = uint32_t(i - lo);
        }
        // deferred records: retry until their predecessors finish; help with
        // the chunk queue meanwhile (chunks never wait, so this always progresses)
        int cur = 0;
        for (;;) {
          __syncthreads();
          const uint32_t nd = sh.ndef[cur];
          if (nd == 0) break;
          if (threadIdx.x == 0) sh.ndef[cur ^ 1] = 0;
          __syncthreads();
          for (uint32_t j = threadIdx.x; j < nd; j += kFreqThreads) {
            const uint32_t off = sh.def[cur][j];
            if (!do_record(q, sh, c, sa, lo + off, k, t, rank, gen))
              sh.def[cur ^ 1][atomicAdd(&sh.ndef[cur ^ 1], 1u)] = off;
          }
          __syncthreads();
          if (sh.ndef[cur ^ 1] == nd) {                 // no progress
            __syncthreads();
            if (threadIdx.x == 0) sh.kind = claim_chunk(q, &sh.work) ? 2 : 0;
            __syncthreads();
            if (sh.kind == 2) {
              sa.flush(sh.blk, q.acc);
              run_chunk(q, sh, sh.work, gen);
            } else if (threadIdx.x == 0) {
              __nanosleep(512);
            }
          }
          cur ^= 1;
        }
        sa.flush(sh.blk, q.acc);
      }
      blk_flush(sh.blk, q.acc);
      __threadfence();
      __syncthreads();
      if (threadIdx.x == 0) atomicSub(q.seg_left + k, 1u);
      lo = hi;
    }
    if (threadIdx.x == 0) {
      __threadfence();
      atomicAdd(&ctl->tiles_done, 1ull);
    }
  }
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

int launch_frequency(const FreqParams& q, int num_sms, cudaStream_t s) {
  if (q.a.n == 0) return 0;
  cudaMemsetAsync(q.ctl, 0, sizeof(FreqCtl), s);
  cudaMemsetAsync(q.run_start, 0xFF, 8 * (uint64_t(q.a.n_api) + 1), s);
  uint64_t b = (q.a.n + 255) / 256;
  if (b > uint64_t(num_sms) * 8) b = uint64_t(num_sms) * 8;
  freq_scan_kernel<<<(unsigned)b, 256, 0, s>>>(q);
  freq_plan_kernel<<<1, 1024, 0, s>>>(q);
  freq_main_kernel<<<num_sms * 2, kFreqThreads, 0, s>>>(q);
  return 3;
}

int launch_frequency_reduce(const FreqReduceParams& q, int num_sms, cudaStream_t s) {
  if (q.n_obj == 0) return 0;
  uint64_t b = (q.n_obj + 255) / 256;
  if (b > uint64_t(num_sms) * 8) b = uint64_t(num_sms) * 8;
  frequency_reduce_kernel<<<(unsigned)b, 256, 0, s>>>(q);
  return 1;
}

}  // namespace drgpum
