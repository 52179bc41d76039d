// NEXT-2 non-uniform access frequency (Def 3.9; §5.2
// l.271; fn 3 l.222 -- coefficient of variation).
//
// The paper keeps, per data object, a hashmap element -> access frequency,
// zeroes it when a GPU API that will access the object starts, counts every
// instrumented access of that API, and when the API finishes tests the
// variance of the frequencies.  Reading R22: the statistics run
// over the elements the API touched; CV is the population coefficient of
// variation; NUAF at API A iff CV > X (20%), exactly
// (n*S2 - S1^2) * 100^2 > X^2 * S1^2, with n = elements A touched, S1 = sum
// of their frequencies, S2 = sum of their squares -- per (object, API) slot.
//
// B200 version, sort-based (no hash tables, no dependent atomics):
//   1. freq_events_kernel: every attributed record is the interval
//      [g0, g1] of global element indices it touches; consecutive records of
//      a warp that touch adjacent, disjoint intervals of one object in one
//      API (sequential sweeps) are merged into one interval first.  Each
//      interval becomes two 64-bit keys (rank << pos_bits) | 4*g0 (start)
//      and (rank << pos_bits) | 4*g1 + 2 (end), a single-element interval
//      ONE key (rank << pos_bits) | 4*g + 1 (point); rank = access-API rank
//      (DRGPUM_FQ_POINTS=0: 2*g0 and 2*g1 + 1, no points).
//   2. An LSD radix sort (8-bit digits, stable: tile histograms, a
//      digit-major exclusive scan, a tile-local stable ranking through shared
//      memory and coalesced stores) orders the keys by (API, element).
//      Passes whose digit is the same for every key are skipped.
//   3. The sweep: a scan of +1 (start) / -1 (end) gives, after key i, the
//      number c of intervals covering the elements between key i and key
//      i+1 -- [ceil(p_i/2), ceil(p_{i+1}/2)) -- i.e. the access frequency of
//      each of those len elements within that API.  Each such run adds
//      (len, c*len, c*c*len) to (n, S1, S2) of its (object, API) slot
//      (intervals never span objects or APIs, so runs with c > 0 do not
//      either; every API's intervals are balanced, so no segmented scan is
//      needed).  Points do not change the count; the last of p equal point
//      keys adds the p extra accesses of its element: (c == 0, p, 2cp + p^2).
//   4. The call's last API may continue in the next call (records are in
//      timestamp order across calls): its sorted keys are carried to the
//      front of the other key buffer and sorted together with the next
//      call's; a query sweeps the carried keys into a copy of the sums.
#include "internal.cuh"

namespace drgpum {

#define FULL_MASK 0xFFFFFFFFu
constexpr int kFT = 256;                       // threads per block, every kernel here
constexpr uint32_t kSweepItems = 8;            // keys per thread in the sweep
constexpr uint32_t kSweepChunk = kFT * kSweepItems;
constexpr uint32_t kSweepSample = 2048;        // object bases staged per block for the sweep's search
#ifndef DRGPUM_FQ_ONESWEEP
#define DRGPUM_FQ_ONESWEEP 1   // one-sweep radix passes; digit totals counted where the keys are written
#endif
constexpr uint32_t kBins = 1u << kFreqRadixBits;  // digit values per radix pass
constexpr uint32_t kBPT = kBins / kFT;            // bins per thread
static_assert(kBins % kFT == 0, "bins are spread evenly over the threads");

__device__ __forceinline__ uint32_t ts_of(const AttrParams& p, uint64_t i) { return __ldcs(&p.recs[i].w) & 0x7FFFFFFFu; }

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

// A lane's cached object.
struct LaneObj {
  uint64_t base = 0, size = 0, eb = 0;
  uint32_t ta = 0, tf = 0, shift = 0, obj = kNone;
};

// the global element interval [g0, g1] record i touches, false if it touches
// no live object (or is malformed); c caches the object between records
__device__ __forceinline__ bool resolve(const FreqParams& q, const uint64_t* l1, LaneObj& c, const uint4& r,
                                        uint32_t t, uint64_t& g0, uint64_t& g1) {
  const AttrParams& p = q.a;
  const uint64_t addr = (uint64_t(r.y) << 32) | r.x;
  const uint32_t size = r.z;
  if (size == 0 || addr > ~0ull - size) return false;
  if (!(addr - c.base < c.size && t > c.ta && t < c.tf)) {
    const uint32_t o = freq_find(p, l1, addr, t);
    if (o == kNone) return false;
    const DevObj d = p.objs[o];
    if (t >= d.t_free) return false;
    c.base = d.base; c.size = d.end - d.base; c.ta = d.t_alloc; c.tf = d.t_free;
    c.shift = d.shift; c.obj = o; c.eb = q.elem_base[o];
  }
  const uint64_t off = addr - c.base, end = min(off + size, c.size);
  g0 = c.eb + (off >> c.shift);
  g1 = c.eb + ((end - 1) >> c.shift);
  return true;
}

__device__ __forceinline__ uint64_t* keys_buf(const FreqParams& q, uint32_t which) {
  return which ? q.keys1 : q.keys0;
}
// buffer holding the keys before radix pass d (skipped passes do not flip)
__device__ __forceinline__ uint32_t buf_before(const FreqParams& q, uint32_t d) {
  uint32_t b = uint32_t(q.ctl[1]);
  for (uint32_t k = 0; k < d; ++k) b ^= q.ctl[8 + k] ? 0u : 1u;
  return b;
}
__device__ __forceinline__ unsigned long long* digit_totals(const FreqParams& q, uint32_t d) {
  return q.ctl + kFreqCtlTot + uint64_t(d) * kBins;
}
__device__ __forceinline__ uint64_t n_keys(const FreqParams& q) {
  const unsigned long long n = q.ctl[0];
  return n < q.cap ? n : q.cap;
}



// ---------------------------------------------------------------- 1. events
// Every pass's digit totals, counted where the keys are written (the event
// kernel, and the carry kernel for the carried keys): per-block shared
// histograms, flushed once per block.
// Digit totals: the event and carry kernels count digit 0 only; one-sweep
// pass d counts digit d + 1 of the keys it ranks (a skipped pass reads the
// keys for it), so the event kernel -- issue-bound -- does one shared atomic
// per key instead of one per pass (0: every digit in the event kernel).
#ifndef DRGPUM_FQ_COUNT_NEXT
#define DRGPUM_FQ_COUNT_NEXT 1
#endif
constexpr bool kFreqCountDigits = DRGPUM_FQ_ONESWEEP && DRGPUM_FQ_COUNT_NEXT;
constexpr uint32_t kHistDigits = kFreqCountDigits ? 1 : kFreqMaxDigits;   // digits counted by events / carry
struct DigitHist {
  uint32_t h[kHistDigits][kBins];
  __device__ void zero() {
    for (uint32_t i = threadIdx.x; i < kHistDigits * kBins; i += blockDim.x) h[i / kBins][i % kBins] = 0;
  }
  __device__ void add(uint64_t key, uint32_t nd) {
    for (uint32_t d = 0; d < nd; ++d) atomicAdd(&h[d][uint32_t(key >> (kFreqRadixBits * d)) & (kBins - 1)], 1u);
  }
  __device__ void flush(const FreqParams& q) {
    for (uint32_t i = threadIdx.x; i < min(q.n_digits, kHistDigits) * kBins; i += blockDim.x) {
      const uint32_t v = h[i / kBins][i % kBins];
      if (v) atomicAdd(q.ctl + kFreqCtlTot + i, (unsigned long long)v);
    }
  }
};

// Keys are staged per warp in shared memory and flushed 256 at a time with
// ONE atomic on the global key count (a per-tile atomic on that single
// address serialised the kernel: 3e6 same-address atomics on C2).
constexpr uint32_t kEvBuf = 256;
__device__ __forceinline__ void ev_flush(const FreqParams& q, uint64_t* out, const uint64_t* buf, uint32_t cnt,
                                         int lane, DigitHist& dh) {
  // per-lane shared atomics: a warp vote (on every digit or only on the
  // mostly uniform high digits) or a MATCH.ANY first measured slower --
  // events 1.12 -> 1.6-2.05 ms on C2
  if (DRGPUM_FQ_ONESWEEP)
    for (uint32_t j = lane; j < cnt; j += 32) dh.add(buf[j], kFreqCountDigits ? 1u : q.n_digits);
  unsigned long long base = 0;
  if (lane == 0 && cnt) base = atomicAdd(&q.ctl[0], (unsigned long long)cnt);
  base = __shfl_sync(FULL_MASK, base, 0);
  if (!cnt) return;
  if (base + cnt > q.cap) {                          // capacity exceeded: flagged, results invalid
    if (lane == 0) atomicOr(q.state, 2u);
    return;
  }
  for (uint32_t j = lane; j < cnt; j += 32) out[base + j] = buf[j];
}

__global__ void __launch_bounds__(kFT) freq_events_kernel(const __grid_constant__ FreqParams q) {
  __shared__ uint64_t s_l1[kL1MaxKeys];
  __shared__ DigitHist s_dh;
  if (DRGPUM_FQ_ONESWEEP) s_dh.zero();
  __shared__ uint64_t s_ev[kFT / 32][kEvBuf];
  const AttrParams& p = q.a;
  for (uint32_t j = threadIdx.x; j < p.n_l1; j += blockDim.x) s_l1[j] = p.l1[j];
  __syncthreads();
  const int lane = threadIdx.x & 31;
  uint64_t* buf = s_ev[threadIdx.x >> 5];
  uint32_t nbuf = 0;
  uint64_t* out = keys_buf(q, uint32_t(q.ctl[1]));
  // each warp walks one contiguous chunk (lane caches stay on one object)
  const uint64_t nwarps = (uint64_t(gridDim.x) * blockDim.x) >> 5;
  const uint64_t gw = (uint64_t(blockIdx.x) * blockDim.x + threadIdx.x) >> 5;
  const uint64_t chunk = ((p.n + nwarps - 1) / nwarps + 31) / 32 * 32;
  const uint64_t w_lo = min(p.n, gw * chunk), w_hi = min(p.n, w_lo + chunk);
  LaneObj c;
  // timestamp order (across the calls too): the record before this warp's
  // chunk, or the previous call's last timestamp
  uint32_t prev_t = w_lo < w_hi ? (w_lo ? ts_of(p, w_lo - 1) : (q.state[1] ? q.state[1] - 1u : 0u)) : 0u;
  bool unsorted = false;
  for (uint64_t i0 = w_lo; i0 < w_hi; i0 += 32) {     // warp-uniform trip count
    const uint64_t i = i0 + lane;
    bool valid = false;
    uint64_t g0 = 0, g1 = 0;
    uint32_t rank = kNone;
    const uint4 rec = i < w_hi ? __ldcs(p.recs + i) : make_uint4(0, 0, 0, 0xFFFFFFFFu);   // streamed once
    const uint32_t t = i < w_hi ? (rec.w & 0x7FFFFFFFu) : 0xFFFFFFFFu;
    const uint32_t tq = __shfl_up_sync(FULL_MASK, t, 1);
    unsorted |= i < w_hi && t < (lane ? tq : prev_t);
    prev_t = __shfl_sync(FULL_MASK, t, 31);   // the last lane's (a full tile, or the chunk end)
    if (i < w_hi && t < p.n_api) {
      rank = __ldg(p.acc_rank + t);
      valid = rank != kNone && resolve(q, s_l1, c, rec, t, g0, g1);
    }
    // merge chains of adjacent, disjoint intervals of one object and API
    const uint32_t obj = valid ? c.obj : kNone;
    const uint64_t pg1 = __shfl_up_sync(FULL_MASK, g1, 1);
    const uint32_t prk = __shfl_up_sync(FULL_MASK, rank, 1);
    const uint32_t pob = __shfl_up_sync(FULL_MASK, obj, 1);
    const uint32_t vb = __ballot_sync(FULL_MASK, valid);
    const bool pv = lane > 0 && ((vb >> (lane - 1)) & 1u);
    const bool chain = valid && pv && prk == rank && pob == obj && g0 == pg1 + 1;
    const uint32_t cb = __ballot_sync(FULL_MASK, chain);
    const bool head = valid && !chain;
    const bool tail = valid && (lane == 31 || !((cb >> (lane + 1)) & 1u));
    const uint32_t hb = __ballot_sync(FULL_MASK, head), tb = __ballot_sync(FULL_MASK, tail);
#if DRGPUM_FQ_POINTS
    // a single-element interval is one point key: no end key
    const bool pt = head && tail && g0 == g1;
    const uint32_t eb_ = __ballot_sync(FULL_MASK, tail && !pt);
#else
    const bool pt = false;
    const uint32_t eb_ = tb;
#endif
    const uint32_t cnt = __popc(hb) + __popc(eb_);
    if (!cnt) continue;
    if (nbuf + cnt > kEvBuf) {                       // warp-uniform
      __syncwarp();
      ev_flush(q, out, buf, nbuf, lane, s_dh);
      __syncwarp();
      nbuf = 0;
    }
    const uint32_t lt = (1u << lane) - 1u;
    const uint64_t hi = uint64_t(rank) << q.pos_bits;
    if (head) buf[nbuf + __popc(hb & lt)] = hi | (kFreqPosMul * g0 + (pt ? 1 : 0));
    if (tail && !pt) buf[nbuf + __popc(hb) + __popc(eb_ & lt)] = hi | (kFreqPosMul * g1 + kFreqPosMul / 2);
    nbuf += cnt;
  }
  __syncwarp();
  ev_flush(q, out, buf, nbuf, lane, s_dh);
  if (__any_sync(FULL_MASK, unsorted) && lane == 0) atomicOr(q.state, 1u);
  if (DRGPUM_FQ_ONESWEEP) {
    __syncthreads();
    s_dh.flush(q);
  }
}

// ---------------------------------------------------------------- 2. radix sort
// Lanes holding the same (kFreqRadixBits + 1)-bit value (the top bit = "no
// key"): one ballot per bit.
#ifndef DRGPUM_FQ_MATCH
#define DRGPUM_FQ_MATCH 1   // peers by one MATCH.ANY (0: one ballot per bit; C2 pass 0.81 -> 0.73 ms)
#endif
__device__ __forceinline__ uint32_t peers_of(uint32_t v) {
  if (DRGPUM_FQ_MATCH) return __match_any_sync(FULL_MASK, v);
  uint32_t m = FULL_MASK;
#pragma unroll
  for (int b = 0; b <= int(kFreqRadixBits); ++b) {
    const uint32_t x = __ballot_sync(FULL_MASK, (v >> b) & 1u);
    m &= ((v >> b) & 1u) ? x : ~x;
  }
  return m;
}

// (a) tile histograms of digit d, digit-major: hist[digit * ntiles + tile];
// totals per digit for the skip test
__global__ void __launch_bounds__(kFT) freq_hist_kernel(const __grid_constant__ FreqParams q, uint32_t d) {
  __shared__ uint32_t s_h[kBins];
  const uint64_t n = n_keys(q);
  const uint64_t ntiles = (n + kFreqTileKeys - 1) / kFreqTileKeys;
  const uint64_t* src = keys_buf(q, buf_before(q, d));
  const uint32_t shift = kFreqRadixBits * d;
  const int lane = threadIdx.x & 31;
  constexpr uint32_t kI = kFreqTileKeys / kFT;
  for (uint64_t tile = blockIdx.x; tile < ntiles; tile += gridDim.x) {
#pragma unroll
    for (uint32_t b = 0; b < kBPT; ++b) s_h[threadIdx.x + b * kFT] = 0;
    __syncthreads();
    const uint64_t t0 = tile * kFreqTileKeys;
    uint32_t dk[kI];
#pragma unroll
    for (uint32_t k = 0; k < kI; ++k) {              // all of the tile's loads in flight at once
      const uint64_t idx = t0 + k * kFT + threadIdx.x;
      dk[k] = idx < n ? uint32_t(__ldcs(src + idx) >> shift) & (kBins - 1) : kBins;
    }
#pragma unroll
    for (uint32_t k = 0; k < kI; ++k) {
      // the whole warp on one digit (the high digits of sorted-ish keys):
      // one shared atomic; otherwise one per key (conflicts are rare then)
      const uint32_t d0 = __shfl_sync(FULL_MASK, dk[k], 0);
      if (__all_sync(FULL_MASK, dk[k] == d0)) {
        if (lane == 0 && d0 < kBins) atomicAdd(&s_h[d0], 32u);
      } else if (dk[k] < kBins) {
        atomicAdd(&s_h[dk[k]], 1u);
      }
    }
    __syncthreads();
#pragma unroll
    for (uint32_t b = 0; b < kBPT; ++b) {
      const uint32_t bin = threadIdx.x + b * kFT;
      const uint32_t v = s_h[bin];
      q.hist[uint64_t(bin) * ntiles + tile] = v;
      if (v) atomicAdd(digit_totals(q, d) + bin, (unsigned long long)v);
    }
    __syncthreads();
  }
}

// block-wide exclusive scan of one value per thread (kFT threads)
__device__ __forceinline__ uint32_t block_excl_scan(uint32_t v, uint32_t* s_w, uint32_t& total) {
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  uint32_t x = v;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const uint32_t y = __shfl_up_sync(FULL_MASK, x, o);
    if (lane >= o) x += y;
  }
  if (lane == 31) s_w[w] = x;
  __syncthreads();
  uint32_t before = 0;
  total = 0;
#pragma unroll
  for (int k = 0; k < kFT / 32; ++k) {
    const uint32_t s = s_w[k];
    before += k < w ? s : 0u;
    total += s;
  }
  __syncthreads();
  return before + x - v;
}

// (b') digit offsets of pass d: one block per digit; its global start is the
// sum of the lower digits' totals, then a block scan along its row of tile
// counts (hist is digit-major: the row is contiguous), each thread a
// contiguous segment of the row
__global__ void __launch_bounds__(kFT) freq_offsets_kernel(const __grid_constant__ FreqParams q, uint32_t d) {
  __shared__ uint32_t s_w[kFT / 32];
  __shared__ unsigned long long s_base;
  const uint64_t n = n_keys(q);
  const uint64_t ntiles = (n + kFreqTileKeys - 1) / kFreqTileKeys;
  const uint32_t dg = blockIdx.x;
  if (dg == 0) {                                      // skip the pass if one digit holds every key
    bool hit = n == 0;
    for (uint32_t k = threadIdx.x; k < kBins; k += kFT) hit |= digit_totals(q, d)[k] == n;
    hit = __syncthreads_or(hit);
    if (threadIdx.x == 0) q.ctl[8 + d] = hit ? 1ull : 0ull;
  }
  if (threadIdx.x < 32) {
    unsigned long long b = 0;
    for (uint32_t k = threadIdx.x; k < dg; k += 32) b += digit_totals(q, d)[k];
#pragma unroll
    for (int o = 16; o; o >>= 1) b += __shfl_xor_sync(FULL_MASK, b, o);
    if (threadIdx.x == 0) s_base = b;
  }
  const uint32_t* row = q.hist + uint64_t(dg) * ntiles;
  uint32_t* orow = q.offs + uint64_t(dg) * ntiles;
  // the row in chunks of kFT * 16 counts through shared memory: coalesced
  // loads / stores, each thread a contiguous 16-count segment for the scan
  constexpr uint32_t kPer = 16, kChunk = kFT * kPer;
  __shared__ uint32_t s_row[kChunk];
  __syncthreads();                                   // s_base
  uint32_t carry = uint32_t(s_base);
  for (uint64_t c0 = 0; c0 < ntiles; c0 += kChunk) {
#pragma unroll
    for (uint32_t j = 0; j < kPer; ++j) {
      const uint64_t i = c0 + j * kFT + threadIdx.x;
      s_row[j * kFT + threadIdx.x] = i < ntiles ? row[i] : 0u;
    }
    __syncthreads();
    uint32_t v[kPer], sum = 0;
#pragma unroll
    for (uint32_t j = 0; j < kPer; ++j) { v[j] = s_row[threadIdx.x * kPer + j]; sum += v[j]; }
    uint32_t tot;
    uint32_t run = carry + block_excl_scan(sum, s_w, tot);
#pragma unroll
    for (uint32_t j = 0; j < kPer; ++j) { s_row[threadIdx.x * kPer + j] = run; run += v[j]; }
    __syncthreads();
#pragma unroll
    for (uint32_t j = 0; j < kPer; ++j) {
      const uint64_t i = c0 + j * kFT + threadIdx.x;
      if (i < ntiles) orow[i] = s_row[j * kFT + threadIdx.x];
    }
    carry += tot;
    __syncthreads();
  }
}

// (c) one block: exclusive scan of part[0, nb) in place (mode 0: the radix
// digit-offset blocks of pass d; mode 1: the sweep chunks of [0, split),
// signed sums)
__global__ void __launch_bounds__(1024) freq_part_scan_kernel(const __grid_constant__ FreqParams q, uint32_t mode,
                                                              uint32_t d) {
  __shared__ long long s_w[32];
  uint64_t nb;
  if (mode == 0) {
    if (q.ctl[8 + d]) return;
    const uint64_t n = n_keys(q);
    const uint64_t ntiles = (n + kFreqTileKeys - 1) / kFreqTileKeys;
    nb = (uint64_t(kBins) * ntiles + kFreqScanItems - 1) / kFreqScanItems;
  } else {
    nb = (q.ctl[2] + kSweepChunk - 1) / kSweepChunk;
  }
  // thread t scans a contiguous segment: its sum, one block scan of the
  // sums, then the segment's exclusive prefixes (one round instead of
  // nb / 1024 block-wide rounds)
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  const uint64_t seg = (nb + blockDim.x - 1) / blockDim.x;
  const uint64_t i0 = min(nb, uint64_t(threadIdx.x) * seg), i1 = min(nb, i0 + seg);
  auto val = [&](uint64_t i) { return mode == 0 ? (long long)q.part[i] : (long long)(int32_t)q.part[i]; };
  long long v = 0;
  for (uint64_t i = i0; i < i1; ++i) v += val(i);
  long long x = v;
  for (int o = 1; o < 32; o <<= 1) {
    const long long y = __shfl_up_sync(FULL_MASK, x, o);
    if (lane >= o) x += y;
  }
  if (lane == 31) s_w[w] = x;
  __syncthreads();
  long long run = x - v;
  for (int k = 0; k < w; ++k) run += s_w[k];
  for (uint64_t i = i0; i < i1; ++i) {
    const long long e = val(i);
    q.part[i] = uint32_t(run);
    run += e;
  }
}

// (d) stable scatter of pass d.  Tile = 4096 keys; warp w ranks its 512
// keys [512w, 512w+512) in 16 rounds of 32 (key order = round-major, lane
// minor) against a per-warp digit counter -- no block barrier inside; one
// block-wide combine turns the warps' digit counts into per-warp offsets;
// keys go to shared memory in digit order and leave it run by run.
__global__ void __launch_bounds__(kFT) freq_scatter_kernel(const __grid_constant__ FreqParams q, uint32_t d) {
  __shared__ uint64_t s_keys[kFreqTileKeys];
  __shared__ uint16_t s_wc[kFT / 32][kBins];          // per-warp digit counts, then offsets (<= 4096)
  __shared__ uint32_t s_start[kBins], s_goff[kBins], s_w[kFT / 32];
  if (q.ctl[8 + d]) return;                          // every key has the same digit: pass skipped
  const uint64_t n = n_keys(q);
  const uint64_t ntiles = (n + kFreqTileKeys - 1) / kFreqTileKeys;
  const uint32_t src_b = buf_before(q, d);
  const uint64_t* src = keys_buf(q, src_b);
  uint64_t* dst = keys_buf(q, src_b ^ 1u);
  const uint32_t shift = kFreqRadixBits * d;
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const uint32_t lt = (1u << lane) - 1u;
  constexpr uint32_t kR = kFreqTileKeys / kFT;       // 16 rounds of 32 keys per warp
  uint16_t* wc = s_wc[warp];
  for (uint64_t tile = blockIdx.x; tile < ntiles; tile += gridDim.x) {
    // the tile's digit counts (thread t: bins t*kBPT ..) -> local starts and global offsets
    uint32_t cnt[kBPT], csum = 0;
#pragma unroll
    for (uint32_t b = 0; b < kBPT; ++b) {
      const uint64_t e = uint64_t(threadIdx.x * kBPT + b) * ntiles + tile;
      cnt[b] = q.hist[e];
      s_goff[threadIdx.x * kBPT + b] = q.offs[e];
      csum += cnt[b];
    }
    uint32_t tot;
    uint32_t st = block_excl_scan(csum, s_w, tot);   // (syncs: the previous tile is written out)
#pragma unroll
    for (uint32_t b = 0; b < kBPT; ++b) { s_start[threadIdx.x * kBPT + b] = st; st += cnt[b]; }
#pragma unroll
    for (uint32_t k = 0; k < kBins / 32; ++k) wc[lane + 32 * k] = 0;
    __syncwarp();
    const uint64_t w0 = tile * kFreqTileKeys + uint64_t(warp) * (kR * 32);
    uint64_t kr[kR];
#pragma unroll
    for (uint32_t r = 0; r < kR; ++r) {              // all of the warp's loads in flight at once
      const uint64_t idx = w0 + r * 32 + lane;
      kr[r] = idx < n ? __ldcs(src + idx) : ~0ull;
    }
    uint32_t rank[kR];
#pragma unroll
    for (uint32_t r = 0; r < kR; ++r) {
      const bool valid = kr[r] != ~0ull;
      const uint32_t dg = valid ? uint32_t(kr[r] >> shift) & (kBins - 1) : kBins;
      const uint32_t d0 = __shfl_sync(FULL_MASK, dg, 0);
      if (__all_sync(FULL_MASK, dg == d0)) {          // one digit for the round (common on high digits)
        if (d0 < kBins) {
          rank[r] = wc[d0] + uint32_t(lane);
          __syncwarp();
          if (lane == 0) wc[d0] = uint16_t(wc[d0] + 32u);
        }
      } else {
        const uint32_t peers = peers_of(dg);
        if (valid) rank[r] = wc[dg] + __popc(peers & lt);
        __syncwarp();
        if (valid && (peers & lt) == 0) wc[dg] = uint16_t(wc[dg] + __popc(peers));
      }
      __syncwarp();
    }
    __syncthreads();
    // per digit: exclusive prefix of the warps' counts
#pragma unroll
    for (uint32_t b = 0; b < kBPT; ++b) {
      const uint32_t bin = threadIdx.x + b * kFT;
      uint32_t run = 0;
#pragma unroll
      for (int w = 0; w < kFT / 32; ++w) {
        const uint32_t v = s_wc[w][bin];
        s_wc[w][bin] = uint16_t(run);
        run += v;
      }
    }
    __syncthreads();
#pragma unroll
    for (uint32_t r = 0; r < kR; ++r) {
      if (kr[r] == ~0ull) continue;
      const uint32_t dg = uint32_t(kr[r] >> shift) & (kBins - 1);
      s_keys[s_start[dg] + wc[dg] + rank[r]] = kr[r];
    }
    __syncthreads();
    const uint64_t t0 = tile * kFreqTileKeys;
    const uint32_t tn = uint32_t(min(uint64_t(kFreqTileKeys), n - t0));
    for (uint32_t j = threadIdx.x; j < tn; j += kFT) {
      const uint64_t key = s_keys[j];
      const uint32_t dg = uint32_t(key >> shift) & (kBins - 1);
      dst[s_goff[dg] + (j - s_start[dg])] = key;
    }
    __syncthreads();   // s_keys / s_goff / s_start are rewritten by the next tile
  }
}

// ---- one-sweep form (default): every pass's digit totals counted where the
// keys were written (event kernel, carry kernel), then ONE kernel per pass: tiles taken in order from a ticket,
// ranked as above, their digit counts published and the exclusive prefix over
// the previous tiles found by decoupled look-back (flag A: the tile's own
// count, flag P: the inclusive prefix), so no per-pass histogram kernel and
// no offset scan.
// Look-back status per (tile, digit): flag A = the tile's own count, flag P =
// inclusive prefix, 30-bit value.  Two status arrays alternate between the
// passes (hist for even, offs for odd passes; offs is free in this form):
// pass d clears, tile by tile, the rows pass d + 1 will use, so only the
// first pass of a sort needs a memset (a u64 status tagged with a pass epoch
// and no clearing measured slower: 0.73 -> 0.84 ms per pass on C2).
constexpr uint32_t kFlagA = 1u << 30, kFlagP = 1u << 31, kValMask = kFlagA - 1;

// skip flags of every pass (a pass whose digit is the same for every key)
__global__ void __launch_bounds__(kFT) freq_skip_kernel(const __grid_constant__ FreqParams q) {
  const uint64_t n = n_keys(q);
  for (uint32_t d = 0; d < q.n_digits; ++d) {
    bool hit = n == 0;
    for (uint32_t k = threadIdx.x; k < kBins; k += kFT) hit |= digit_totals(q, d)[k] == n;
    hit = __syncthreads_or(hit);
    if (threadIdx.x == 0) q.ctl[8 + d] = hit ? 1ull : 0ull;
  }
}

#ifndef DRGPUM_FQ_ATOMRANK
#define DRGPUM_FQ_ATOMRANK 1
#endif
#ifndef DRGPUM_FQ_MINB
#define DRGPUM_FQ_MINB 4   // blocks per SM of the one-sweep pass (register cap 64; C2: 0.755 -> 0.722 ms vs 3)
#endif
__global__ void __launch_bounds__(kFT, DRGPUM_FQ_MINB) freq_onesweep_kernel(const __grid_constant__ FreqParams q, uint32_t d) {
  __shared__ uint64_t s_keys[kFreqTileKeys];
  __shared__ uint16_t s_wc[kFT / 32][kBins];          // per-warp digit counts, then offsets (<= 4096)
  __shared__ uint32_t s_start[kBins], s_goff[kBins], s_w[kFT / 32];
  __shared__ uint32_t s_tile;
  __shared__ uint32_t s_nx[kBins];                   // digit d + 1 of this block's keys (kFreqCountDigits)
  const uint64_t n = n_keys(q);
  const uint64_t ntiles = (n + kFreqTileKeys - 1) / kFreqTileKeys;
  volatile uint32_t* status = (d & 1) ? q.offs : q.hist;   // [tile][bin]
  uint32_t* status_next = (d & 1) ? q.hist : q.offs;       // pass d + 1's, cleared here
  const bool count_next = kFreqCountDigits && d + 1 < q.n_digits;
  bool skip;
  if (kFreqCountDigits) {   // every key has the same digit d (a total equals n): pass skipped
    for (uint32_t k = threadIdx.x; k < kBins; k += kFT) s_nx[k] = 0;
    bool hit = n == 0;
    for (uint32_t k = threadIdx.x; k < kBins; k += kFT) hit |= digit_totals(q, d)[k] == n;
    skip = __syncthreads_or(hit);
    if (blockIdx.x == 0 && threadIdx.x == 0) q.ctl[8 + d] = skip ? 1ull : 0ull;
  } else {
    skip = q.ctl[8 + d] != 0;
  }
  const uint32_t src_b = buf_before(q, d);
  if (skip) {
    for (uint64_t i = uint64_t(blockIdx.x) * kFT + threadIdx.x; i < ntiles * kBins; i += uint64_t(gridDim.x) * kFT)
      status_next[i] = 0;
    if (count_next) {   // the next pass's digit totals from the unmoved keys
      const uint64_t* kk = keys_buf(q, src_b);
      for (uint64_t i = uint64_t(blockIdx.x) * kFT + threadIdx.x; i < n; i += uint64_t(gridDim.x) * kFT)
        atomicAdd(&s_nx[uint32_t(kk[i] >> (kFreqRadixBits * (d + 1))) & (kBins - 1)], 1u);
      __syncthreads();
      for (uint32_t k = threadIdx.x; k < kBins; k += kFT)
        if (s_nx[k]) atomicAdd(digit_totals(q, d + 1) + k, (unsigned long long)s_nx[k]);
    }
    return;
  }
  const uint64_t* src = keys_buf(q, src_b);
  uint64_t* dst = keys_buf(q, src_b ^ 1u);
  const uint32_t shift = kFreqRadixBits * d;
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const uint32_t lt = (1u << lane) - 1u;
  constexpr uint32_t kR = kFreqTileKeys / kFT;
  uint16_t* wc = s_wc[warp];
  uint32_t gstart[kBPT];   // global digit starts of this thread's bins (exclusive scan of the totals)
  {
    const unsigned long long* tot = digit_totals(q, d);
    uint32_t c[kBPT], cs = 0;
#pragma unroll
    for (uint32_t b = 0; b < kBPT; ++b) { c[b] = uint32_t(tot[threadIdx.x * kBPT + b]); cs += c[b]; }
    uint32_t all;
    uint32_t st = block_excl_scan(cs, s_w, all);
#pragma unroll
    for (uint32_t b = 0; b < kBPT; ++b) { gstart[b] = st; st += c[b]; }
  }
  for (;;) {
    if (threadIdx.x == 0) s_tile = uint32_t(atomicAdd(&q.ctl[16 + d], 1ull));
    __syncthreads();
    const uint64_t tile = s_tile;
    if (tile >= ntiles) break;
#pragma unroll
    for (uint32_t k = 0; k < kBins / 32; ++k) wc[lane + 32 * k] = 0;
    __syncwarp();
    const uint64_t w0 = tile * kFreqTileKeys + uint64_t(warp) * (kR * 32);
    uint64_t kr[kR];
#pragma unroll
    for (uint32_t r = 0; r < kR; ++r) {
      const uint64_t idx = w0 + r * 32 + lane;
      kr[r] = idx < n ? __ldcs(src + idx) : ~0ull;
    }
    if (count_next) {
#pragma unroll
      for (uint32_t r = 0; r < kR; ++r)
        if (kr[r] != ~0ull) atomicAdd(&s_nx[uint32_t(kr[r] >> (shift + kFreqRadixBits)) & (kBins - 1)], 1u);
    }
    uint32_t rank[kR];
#if DRGPUM_FQ_ATOMRANK
    // each round's leader adds its peer count to the warp's digit counter with
    // a returning shared atomic (two u16 counters per u32 word) and hands the
    // old value to its peers: no read-modify-write chain through syncwarps,
    // the rounds' atomics pipeline (same-address ones stay in program order)
    uint32_t* wc32 = reinterpret_cast<uint32_t*>(wc);
#pragma unroll
    for (uint32_t r = 0; r < kR; ++r) {
      const bool valid = kr[r] != ~0ull;
      const uint32_t dg = valid ? uint32_t(kr[r] >> shift) & (kBins - 1) : kBins;
      const uint32_t peers = peers_of(dg);
      const int leader = __ffs(peers) - 1;
      const uint32_t sh = (dg & 1u) * 16u;
      uint32_t old = 0;
      if (valid && leader == lane) old = atomicAdd(wc32 + (dg >> 1), uint32_t(__popc(peers)) << sh);
      old = __shfl_sync(FULL_MASK, old, leader);
      rank[r] = ((old >> sh) & 0xFFFFu) + __popc(peers & lt);
    }
    __syncwarp();
#else
#pragma unroll
    for (uint32_t r = 0; r < kR; ++r) {
      const bool valid = kr[r] != ~0ull;
      const uint32_t dg = valid ? uint32_t(kr[r] >> shift) & (kBins - 1) : kBins;
      const uint32_t d0 = __shfl_sync(FULL_MASK, dg, 0);
      if (__all_sync(FULL_MASK, dg == d0)) {
        if (d0 < kBins) {
          rank[r] = wc[d0] + uint32_t(lane);
          __syncwarp();
          if (lane == 0) wc[d0] = uint16_t(wc[d0] + 32u);
        }
      } else {
        const uint32_t peers = peers_of(dg);
        if (valid) rank[r] = wc[dg] + __popc(peers & lt);
        __syncwarp();
        if (valid && (peers & lt) == 0) wc[dg] = uint16_t(wc[dg] + __popc(peers));
      }
      __syncwarp();
    }
#endif
    __syncthreads();
    // per digit: the tile's count, the warps' offsets, publish, look back
    uint32_t cnt[kBPT], csum = 0;
#pragma unroll
    for (uint32_t b = 0; b < kBPT; ++b) {
      const uint32_t bin = threadIdx.x * kBPT + b;
      uint32_t run = 0;
#pragma unroll
      for (int w = 0; w < kFT / 32; ++w) {
        const uint32_t v = s_wc[w][bin];
        s_wc[w][bin] = uint16_t(run);
        run += v;
      }
      cnt[b] = run;
      csum += run;
      __stcg(const_cast<uint32_t*>(status) + tile * kBins + bin, (tile == 0 ? kFlagP : kFlagA) | run);
      status_next[tile * kBins + bin] = 0;
    }
    uint32_t tsum;
    uint32_t st = block_excl_scan(csum, s_w, tsum);
#pragma unroll
    for (uint32_t b = 0; b < kBPT; ++b) {
      const uint32_t bin = threadIdx.x * kBPT + b;
      s_start[bin] = st;
      st += cnt[b];
      uint32_t excl = 0;
      for (int64_t pt = int64_t(tile) - 1; pt >= 0;) {   // decoupled look-back
        const uint32_t v = status[uint64_t(pt) * kBins + bin];
        if (v & kFlagP) { excl += v & kValMask; break; }
        if (v & kFlagA) { excl += v & kValMask; --pt; }
      }
      if (tile) __stcg(const_cast<uint32_t*>(status) + tile * kBins + bin, kFlagP | (excl + cnt[b]));
      s_goff[bin] = gstart[b] + excl;
    }
    __syncthreads();
#pragma unroll
    for (uint32_t r = 0; r < kR; ++r) {
      if (kr[r] == ~0ull) continue;
      const uint32_t dg = uint32_t(kr[r] >> shift) & (kBins - 1);
      s_keys[s_start[dg] + wc[dg] + rank[r]] = kr[r];
    }
    __syncthreads();
    const uint32_t tn = uint32_t(min(uint64_t(kFreqTileKeys), n - tile * kFreqTileKeys));
    for (uint32_t j = threadIdx.x; j < tn; j += kFT) {
      const uint64_t key = s_keys[j];
      const uint32_t dg = uint32_t(key >> shift) & (kBins - 1);
      dst[s_goff[dg] + (j - s_start[dg])] = key;
    }
    __syncthreads();
  }
  if (count_next)   // (the loop's last __syncthreads: every count is in)
    for (uint32_t k = threadIdx.x; k < kBins; k += kFT)
      if (s_nx[k]) atomicAdd(digit_totals(q, d + 1) + k, (unsigned long long)s_nx[k]);
}

// ---------------------------------------------------------------- 3. sweep
// split = first key of the call's last API (carried to the next call);
// queries (mode 1) sweep every key
__global__ void freq_split_kernel(const __grid_constant__ FreqParams q, uint32_t mode) {
  const uint64_t n = n_keys(q);
  if (q.state[0] & 2u) { q.ctl[2] = 0; return; }     // capacity exceeded: nothing is valid
  if (mode == 1 || n == 0) { q.ctl[2] = n; return; }
  const uint64_t* k = keys_buf(q, buf_before(q, q.n_digits));
  const uint64_t target = (k[n - 1] >> q.pos_bits) << q.pos_bits;
  uint64_t lo = 0, hi = n;
  while (lo < hi) { const uint64_t m = (lo + hi) / 2; if (k[m] < target) lo = m + 1; else hi = m; }
  q.ctl[2] = lo;
}

// +1 start, -1 end, 0 point (the point's count is added at its element only)
__device__ __forceinline__ int ev_sign(uint64_t key) {
  return DRGPUM_FQ_POINTS ? 1 - int(key & 3u) : ((key & 1ull) ? -1 : 1);
}
// the element from which the count after this key applies: start g -> g,
// point g -> g (no change there), end g -> g + 1
__device__ __forceinline__ uint64_t ev_x(uint64_t pos) {
  return DRGPUM_FQ_POINTS ? (pos + 2) >> 2 : (pos + 1) >> 1;
}
__device__ __forceinline__ bool ev_point(uint64_t key) { return DRGPUM_FQ_POINTS && (key & 3u) == 1; }

// per chunk of kSweepChunk keys of [0, split): sum of the +1 / -1 events
__global__ void __launch_bounds__(kFT) freq_sweep_sum_kernel(const __grid_constant__ FreqParams q) {
  __shared__ uint32_t s_w[kFT / 32];
  const uint64_t split = q.ctl[2];
  const uint64_t* k = keys_buf(q, buf_before(q, q.n_digits));
  const uint64_t nb = (split + kSweepChunk - 1) / kSweepChunk;
  for (uint64_t b = blockIdx.x; b < nb; b += gridDim.x) {
    const uint64_t c0 = b * kSweepChunk;
    int s = 0;
#pragma unroll
    for (uint32_t j = 0; j < kSweepItems; ++j) {     // coalesced: the order does not matter for a sum
      const uint64_t i = c0 + j * kFT + threadIdx.x;
      if (i < split) s += ev_sign(__ldcs(k + i));
    }
    uint32_t total;
    block_excl_scan(uint32_t(s), s_w, total);
    if (threadIdx.x == 0) q.part[b] = total;
  }
}

struct SlotSum {
  uint64_t slot = ~0ull, n = 0, s1 = 0, s2 = 0;
  __device__ void flush(unsigned long long* acc) {
    if (slot != ~0ull && n) {
      atomicAdd(acc + 3 * slot, (unsigned long long)n);
      atomicAdd(acc + 3 * slot + 1, (unsigned long long)s1);
      atomicAdd(acc + 3 * slot + 2, (unsigned long long)s2);
    }
    n = s1 = s2 = 0;
  }
};

// the runs: from key i (count c after it) to key i+1, len = ceil(p_{i+1}/2)
// - ceil(p_i/2) elements with frequency c in the API of key i
__global__ void __launch_bounds__(kFT) freq_sweep_kernel(const __grid_constant__ FreqParams q,
                                                         unsigned long long* acc) {
  __shared__ uint32_t s_w[kFT / 32];
  __shared__ uint64_t s_eb[kSweepSample];            // element base of every stride-th object
  __shared__ uint64_t s_k[kSweepChunk + kSweepChunk / 8 + 2];   // padded: 1 word per 8
  const uint32_t n_obj = uint32_t(q.n_obj);
  const uint32_t stride = n_obj ? (n_obj + kSweepSample - 1) / kSweepSample : 1u;
  const uint32_t n_samp = (n_obj + stride - 1) / stride;
  for (uint32_t i = threadIdx.x; i < n_samp; i += kFT) s_eb[i] = q.elem_base[uint64_t(i) * stride];
  __syncthreads();
  const uint64_t split = q.ctl[2];
  const uint64_t* k = keys_buf(q, buf_before(q, q.n_digits));
  const uint64_t nb = (split + kSweepChunk - 1) / kSweepChunk;
  const uint64_t pmask = (1ull << q.pos_bits) - 1;
  uint64_t c_lo = 1, c_hi = 0, c_sb = 0;          // cached object's element range, slot base, r_lo
  uint32_t c_rlo = 0;
  SlotSum ss;
  for (uint64_t b = blockIdx.x; b < nb; b += gridDim.x) {
    // the chunk (+ the next key) through shared memory: coalesced loads,
    // then every thread its kSweepItems consecutive keys
    const uint64_t c0 = b * kSweepChunk;
#pragma unroll
    for (uint32_t j = 0; j < kSweepItems; ++j) {
      const uint64_t i = c0 + j * kFT + threadIdx.x;
      const uint32_t li = j * kFT + threadIdx.x;
      s_k[li + (li >> 3)] = i < split ? __ldcs(k + i) : ~0ull;
    }
    if (threadIdx.x == 0) s_k[kSweepChunk + kSweepChunk / 8] = c0 + kSweepChunk < split ? k[c0 + kSweepChunk] : ~0ull;
    __syncthreads();
    uint64_t kk[kSweepItems + 1];
    int s = 0;
#pragma unroll
    for (uint32_t j = 0; j <= kSweepItems; ++j) {
      const uint32_t li = threadIdx.x * kSweepItems + j;   // li >> 3 == thread (+1 for the next key)
      kk[j] = s_k[li + (li >> 3)];
    }
    __syncthreads();
#pragma unroll
    for (uint32_t j = 0; j < kSweepItems; ++j) if (kk[j] != ~0ull) s += ev_sign(kk[j]);
    uint32_t total;
    int c = int(q.part[b]) + int(block_excl_scan(uint32_t(s), s_w, total));
    auto locate = [&](uint64_t x0) {                 // object of element x0: shared sample, then global
      if (x0 >= c_lo && x0 < c_hi) return;
      uint32_t a = 0, bb = n_samp;
      while (bb - a > 1) { const uint32_t m = (a + bb) >> 1; if (s_eb[m] <= x0) a = m; else bb = m; }
      uint32_t lo = a * stride, hi = min(n_obj, lo + stride);
      while (hi - lo > 1) { const uint32_t m = (lo + hi) >> 1; if (q.elem_base[m] <= x0) lo = m; else hi = m; }
      const DevObj dv = q.a.objs[lo];
      c_lo = q.elem_base[lo];
      c_hi = c_lo + ((dv.end - dv.base) >> dv.shift);
      c_sb = q.slot_base[lo];
      c_rlo = dv.r_lo;
    };
#pragma unroll
    for (uint32_t j = 0; j < kSweepItems; ++j) {
      if (kk[j] == ~0ull) break;
      c += ev_sign(kk[j]);
      if (ev_point(kk[j]) && kk[j + 1] != kk[j]) {
        // last of a run of p equal point keys: element g has count c + p
        // (c = the intervals covering it, already in its run): n + [c == 0],
        // S1 + p, S2 + (c + p)^2 - c^2
        // (the key before it from registers, earlier ones -- long runs -- from L2)
        uint64_t p = 1;
        const uint64_t gi = c0 + uint64_t(threadIdx.x) * kSweepItems + j;   // global index of key j
        if (gi > 0 && (j > 0 ? kk[j - 1] : k[gi - 1]) == kk[j]) {
          p = 2;
          while (p <= gi && k[gi - p] == kk[j]) ++p;
        }
        const uint64_t g = (kk[j] & pmask) >> 2;
        locate(g);
        const uint64_t slot = c_sb + ((kk[j] >> q.pos_bits) - c_rlo);
        if (slot != ss.slot) { ss.flush(acc); ss.slot = slot; }
        const uint64_t cu = uint64_t(c);
        ss.n += cu == 0 ? 1 : 0;
        ss.s1 += p;
        ss.s2 += 2 * cu * p + p * p;
      }
      if (c <= 0 || kk[j + 1] == ~0ull) continue;   // c > 0: the next key belongs to the same API
      const uint64_t x0 = ev_x(kk[j] & pmask), x1 = ev_x(kk[j + 1] & pmask);
      if (x1 <= x0) continue;
      const uint64_t len = x1 - x0;
      locate(x0);
      const uint64_t slot = c_sb + ((kk[j] >> q.pos_bits) - c_rlo);
      if (slot != ss.slot) { ss.flush(acc); ss.slot = slot; }
      const uint64_t cu = uint64_t(c);
      ss.n += len;
      ss.s1 += cu * len;
      ss.s2 += cu * cu * len;
    }
  }
  ss.flush(acc);
}

// ---------------------------------------------------------------- 4. carry
__global__ void __launch_bounds__(kFT) freq_carry_kernel(const __grid_constant__ FreqParams q) {
  __shared__ DigitHist s_dh;                          // the carried keys count toward the next sort
  if (DRGPUM_FQ_ONESWEEP) s_dh.zero();
  __syncthreads();
  const uint64_t n = n_keys(q), split = q.ctl[2];
  const uint32_t b = buf_before(q, q.n_digits);
  const uint64_t* src = keys_buf(q, b);
  uint64_t* dst = keys_buf(q, b ^ 1u);
  for (uint64_t i = split + uint64_t(blockIdx.x) * blockDim.x + threadIdx.x; i < n;
       i += uint64_t(gridDim.x) * blockDim.x) {
    const uint64_t key = src[i];
    dst[i - split] = key;
    if (DRGPUM_FQ_ONESWEEP) s_dh.add(key, kFreqCountDigits ? 1u : q.n_digits);
  }
  if (DRGPUM_FQ_ONESWEEP) {
    __syncthreads();
    s_dh.flush(q);
  }
}

__global__ void freq_carry_ctl_kernel(const __grid_constant__ FreqParams q) {
  const uint64_t n = n_keys(q), split = q.ctl[2];
  const uint32_t b = buf_before(q, q.n_digits);
  q.ctl[0] = n - split;
  q.ctl[1] = b ^ 1u;
  for (int d = 0; d < 8; ++d) q.ctl[8 + d] = 0;
  if (q.a.n) q.state[1] = ts_of(q.a, q.a.n - 1) + 1u;
}

// ---------------------------------------------------------------- launchers
#ifndef DRGPUM_FQ_GRID
#define DRGPUM_FQ_GRID 4
#endif
static void radix_sort(const FreqParams& q, int num_sms, cudaStream_t s, int& launches) {
  const unsigned g = unsigned(num_sms) * DRGPUM_FQ_GRID;
#if DRGPUM_FQ_ONESWEEP
  // digit totals: counted by the event kernel (and the previous call's carry)
  cudaMemsetAsync(q.ctl + 8, 0, 8 * 16, s);   // skip flags, tickets
  cudaMemsetAsync(q.hist, 0, 4ull * kBins * q.max_tiles, s);   // first pass's look-back status
  if (!kFreqCountDigits) {   // skip flags from the totals (otherwise each pass decides its own)
    freq_skip_kernel<<<1, kFT, 0, s>>>(q);
    launches += 1;
  }
  for (uint32_t d = 0; d < q.n_digits; ++d) {
    freq_onesweep_kernel<<<g, kFT, 0, s>>>(q, d);
    launches += 1;
  }
#else
  cudaMemsetAsync(q.ctl + 8, 0, 8 * (kFreqCtlWords - 8), s);   // skip flags, tickets, totals
  for (uint32_t d = 0; d < q.n_digits; ++d) {
    freq_hist_kernel<<<g, kFT, 0, s>>>(q, d);
    freq_offsets_kernel<<<kBins, kFT, 0, s>>>(q, d);
    freq_scatter_kernel<<<g, kFT, 0, s>>>(q, d);
    launches += 3;
  }
#endif
}

static void sweep(const FreqParams& q, unsigned long long* acc, uint32_t mode, int num_sms, cudaStream_t s,
                  int& launches) {
  const unsigned g = unsigned(num_sms) * 4;
  freq_split_kernel<<<1, 1, 0, s>>>(q, mode);
  freq_sweep_sum_kernel<<<g, kFT, 0, s>>>(q);
  freq_part_scan_kernel<<<1, 1024, 0, s>>>(q, 1, 0);
  freq_sweep_kernel<<<g, kFT, 0, s>>>(q, acc);
  launches += 4;
}

int launch_frequency(const FreqParams& q, int num_sms, cudaStream_t s) {
  if (q.a.n == 0) return 0;
  int launches = 0;
  // one wave: every warp walks one contiguous chunk, so blocks beyond the
  // resident ones would form a second, partial wave (a register cap for 6 or
  // 8 blocks per SM measured slower: 0.93 -> 0.97 / 1.01 ms on C2)
  int ev_occ = 0;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&ev_occ, freq_events_kernel, kFT, 0);
  freq_events_kernel<<<unsigned(num_sms) * unsigned(ev_occ < 1 ? 1 : ev_occ), kFT, 0, s>>>(q);   // also checks the timestamp order
  launches += 1;
  radix_sort(q, num_sms, s, launches);
  sweep(q, q.acc, 0, num_sms, s, launches);
  // the next sort's digit totals start with the carried keys
  cudaMemsetAsync(q.ctl + kFreqCtlTot, 0, 8ull * kFreqMaxDigits * kBins, s);
  freq_carry_kernel<<<unsigned(num_sms) * 4, kFT, 0, s>>>(q);
  freq_carry_ctl_kernel<<<1, 1, 0, s>>>(q);
  return launches + 2;
}

int launch_frequency_query(const FreqParams& q, uint64_t n_slots, int num_sms, cudaStream_t s) {
  int launches = 0;
  if (n_slots) cudaMemcpyAsync(q.acc_q, q.acc, 24 * n_slots, cudaMemcpyDeviceToDevice, s);
  // the carried keys are the sorted tail of the last call: swept as they
  // are, with no radix pass (n_digits = 0 selects the current buffer)
  FreqParams z = q;
  z.n_digits = 0;
  sweep(z, q.acc_q, 1, num_sms, s, launches);
  return launches;
}

// per object: the APIs at which it matches NUAF, and the first of them
// (one warp per object, lanes over its slots)
__global__ void __launch_bounds__(256) frequency_reduce_kernel(const FreqReduceParams q) {
  const int lane = threadIdx.x & 31;
  const uint64_t gw = (uint64_t(blockIdx.x) * blockDim.x + threadIdx.x) >> 5;
  const uint64_t nw = (uint64_t(gridDim.x) * blockDim.x) >> 5;
  using u128 = unsigned __int128;
  for (uint64_t o = gw; o < q.n_obj; o += nw) {
    const uint64_t sb = q.slot_base[o];
    const uint32_t nh = q.n_hit[o], r_lo = q.objs[o].r_lo;
    uint32_t cnt = 0, first_k = 0xFFFFFFFFu;
    for (uint32_t k = lane; k < nh; k += 32) {
      const unsigned long long* a = q.acc + 3 * (sb + k);
      const u128 n = a[0], s1 = a[1], s2 = a[2];
      // CV^2 = (n*S2 - S1^2)/S1^2 > (pct/100)^2
      if (s1 && (n * s2 - s1 * s1) * 10000u > u128(q.pct) * q.pct * s1 * s1) {
        ++cnt;
        first_k = min(first_k, k);
      }
    }
    cnt = __reduce_add_sync(FULL_MASK, cnt);
    first_k = __reduce_min_sync(FULL_MASK, first_k);
    if (lane == 0) {
      q.out_count[o] = cnt;
      q.out_first[o] = first_k == 0xFFFFFFFFu ? kNever : q.acc_ts[r_lo + first_k];
    }
  }
}

int launch_frequency_reduce(const FreqReduceParams& q, int num_sms, cudaStream_t s) {
  if (q.n_obj == 0) return 0;
  uint64_t b = (q.n_obj + 7) / 8;
  if (b > uint64_t(num_sms) * 16) b = uint64_t(num_sms) * 16;
  frequency_reduce_kernel<<<(unsigned)b, 256, 0, s>>>(q);
  return 1;
}

}  // namespace drgpum
