// NEXT-2 non-uniform access frequency (Def 3.9; §5.2
// l.271; fn 3 l.222 -- coefficient of variation).
//
// The paper keeps, per data object, a hashmap element -> access frequency,
// zeroes it when a GPU API that will access the object starts, counts every
// instrumented access of that API, and when the API finishes tests the
// variance of the frequencies.  Reading R22: the statistics run
// over the elements the API touched (the hashmap's cells); CV is the
// population coefficient of variation; NUAF at API A iff CV > X (20%),
// exactly: 25*(n*S2 - S1^2) > S1^2 for X = 20.
//
// B200 version.  One cooperative kernel walks the timestamp-sorted trace one
// API segment at a time (grid barrier between segments).  Each element owns a
// 64-bit cell {API tag, count}; a CAS either continues the count of the
// current API or restarts it (the tag replaces the paper's explicit zeroing,
// which is safe because segments are processed strictly one after another).
// Every increment returns the element's previous count c, so the (object,
// API) sums follow without a second pass: n += (c == 0), S1 += 1,
// S2 += 2c + 1.  Lanes accumulate locally while they stay in one (object, API)
// slot and flush with three 64-bit atomics.  Records wider than 64 elements
// go to a queue that the whole grid expands after the segment's barrier.
#include <cooperative_groups.h>

#include "internal.cuh"

namespace cg = cooperative_groups;

namespace drgpum {

constexpr uint64_t kFreqInline = 64;
constexpr uint64_t kFreqChunk = 4096;

__device__ __forceinline__ uint32_t freq_incr(unsigned long long* cell, uint32_t tag) {
  unsigned long long cur = *reinterpret_cast<volatile unsigned long long*>(cell);
  for (;;) {
    const bool same = uint32_t(cur >> 32) == tag;
    const unsigned long long want = same ? cur + 1 : ((unsigned long long)tag << 32) | 1ull;
    const unsigned long long prev = atomicCAS(cell, cur, want);
    if (prev == cur) return same ? uint32_t(cur) : 0u;
    cur = prev;
  }
}

struct SlotAcc {
  uint64_t slot = ~0ull, n = 0, s1 = 0, s2 = 0;
  __device__ void flush(unsigned long long* acc) {
    if (slot != ~0ull && s1) {
      atomicAdd(acc + 3 * slot, (unsigned long long)n);
      atomicAdd(acc + 3 * slot + 1, (unsigned long long)s1);
      atomicAdd(acc + 3 * slot + 2, (unsigned long long)s2);
    }
    n = s1 = s2 = 0;
  }
  __device__ void add(unsigned long long* acc, uint64_t sl, uint32_t prev) {
    if (sl != slot) { flush(acc); slot = sl; }
    n += prev == 0;
    s1 += 1;
    s2 += 2ull * prev + 1;
  }
};

// object lookup (same index and rules as the attribution kernel)
__device__ __forceinline__ uint32_t freq_find(const AttrParams& p, uint64_t addr, uint32_t ts) {
  if (p.n_seg == 0 || addr < p.l1[0]) return kNone;
  uint32_t lo = 0, hi = p.n_l1;
  while (hi - lo > 1) { const uint32_t m = (lo + hi) >> 1; if (p.l1[m] <= addr) lo = m; else hi = m; }
  uint32_t a = lo * p.l1_stride, b = min(a + p.l1_stride, p.n_seg);
  while (b - a > 1) { const uint32_t m = (a + b) >> 1; if (p.seg_start[m] <= addr) a = m; else b = m; }
  const uint32_t c0 = p.seg_cand_off[a], c1 = p.seg_cand_off[a + 1];
  if (c0 == c1) return kNone;
  uint32_t l = c0, h = c1;
  while (l < h) { const uint32_t m = (l + h) >> 1; if (p.cand[m].t_alloc < ts) l = m + 1; else h = m; }
  return l == c0 ? kNone : p.cand[l - 1].obj;
}

__global__ void __launch_bounds__(256) frequency_kernel(const __grid_constant__ FreqParams q) {
  cg::grid_group g = cg::this_grid();
  const AttrParams& p = q.a;
  const uint64_t tid = uint64_t(blockIdx.x) * blockDim.x + threadIdx.x;
  const uint64_t nth = uint64_t(gridDim.x) * blockDim.x;
  const int lane = threadIdx.x & 31;
  const uint64_t gwarp = tid >> 5, nwarps = nth >> 5;
  auto ts_of = [&](uint64_t i) { return p.recs[i].w & 0x7FFFFFFFu; };
  // the walk needs the trace in API order (within and across calls)
  for (uint64_t i = tid + 1; i < p.n; i += nth)
    if (ts_of(i) < ts_of(i - 1)) atomicOr(q.state, 1u);
  if (tid == 0 && p.n && ts_of(0) < q.state[1]) atomicOr(q.state, 1u);
  g.sync();
  if (*reinterpret_cast<volatile uint32_t*>(q.state)) return;

  uint64_t c_base = 0, c_size = 0, c_eb = 0, c_sb = 0;
  uint32_t c_ta = 0, c_tf = 0, c_rlo = 0, c_shift = 0;
  uint64_t q_done = 0;
  SlotAcc sa;
  for (uint64_t lo = 0; lo < p.n;) {
    const uint32_t t = ts_of(lo);
    uint64_t a = lo, b = p.n;                  // first record with ts > t
    while (a < b) { const uint64_t m = (a + b) >> 1; if (ts_of(m) <= t) a = m + 1; else b = m; }
    const uint64_t hi = a;
    const uint32_t rank = t < p.n_api ? p.acc_rank[t] : kNone;
    if (rank != kNone) {
      const uint32_t tag = rank + 1;
      for (uint64_t i = lo + tid; i < hi; i += nth) {
        const uint4 r = p.recs[i];
        const uint64_t addr = (uint64_t(r.y) << 32) | r.x;
        const uint32_t size = r.z;
        if (size == 0 || addr > ~0ull - size) continue;
        if (!(addr - c_base < c_size && t > c_ta && t < c_tf)) {
          const uint32_t o = freq_find(p, addr, t);
          if (o == kNone) continue;
          const DevObj d = p.objs[o];
          if (t >= d.t_free) continue;
          c_base = d.base; c_size = d.end - d.base; c_ta = d.t_alloc; c_tf = d.t_free;
          c_rlo = d.r_lo; c_shift = d.shift; c_eb = q.elem_base[o]; c_sb = q.slot_base[o];
        }
        const uint64_t off = addr - c_base, end = min(off + size, c_size);
        const uint64_t e0 = off >> c_shift, e1 = (end - 1) >> c_shift;
        const uint64_t slot = c_sb + (rank - c_rlo);
        if (e1 - e0 < kFreqInline) {
          for (uint64_t e = e0; e <= e1; ++e) sa.add(q.acc, slot, freq_incr(q.cells + c_eb + e, tag));
        } else {
          const uint64_t nch = (e1 - e0) / kFreqChunk + 1;
          const unsigned long long s0 = atomicAdd(q.q_count, (unsigned long long)nch);
          for (uint64_t k = 0; k < nch; ++k) {
            const uint64_t l0 = e0 + k * kFreqChunk, h0 = min(e1, l0 + kFreqChunk - 1);
            if (s0 + k < q.q_cap) {
              q.q[s0 + k] = FreqRange{c_eb + l0, c_eb + h0, slot, tag, 0};
            } else {
              for (uint64_t e = l0; e <= h0; ++e) sa.add(q.acc, slot, freq_incr(q.cells + c_eb + e, tag));
            }
          }
        }
      }
      sa.flush(q.acc);
      g.sync();
      const unsigned long long qc_raw = *reinterpret_cast<volatile unsigned long long*>(q.q_count);
      const uint64_t qc = qc_raw < q.q_cap ? qc_raw : q.q_cap;
      if (qc > q_done) {                         // this segment's wide records, whole grid
        for (uint64_t e = q_done + gwarp; e < qc; e += nwarps) {
          const FreqRange fr = q.q[e];
          for (uint64_t x = fr.g_lo + lane; x <= fr.g_hi; x += 32)
            sa.add(q.acc, fr.slot, freq_incr(q.cells + x, fr.tag));
          sa.flush(q.acc);
        }
        q_done = qc;
        g.sync();
      }
    }
    lo = hi;
  }
  if (tid == 0 && p.n) q.state[1] = ts_of(p.n - 1);
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
  cudaMemsetAsync(q.q_count, 0, sizeof(unsigned long long), s);
  static int occ = 0;
  if (!occ) {
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, frequency_kernel, 256, 0);
    if (occ < 1) occ = 1;
    if (occ > 4) occ = 4;
  }
  void* args[] = {const_cast<FreqParams*>(&q)};
  cudaLaunchCooperativeKernel((void*)frequency_kernel, dim3(num_sms * occ), dim3(256), args, 0, s);
  return 1;
}

int launch_frequency_reduce(const FreqReduceParams& q, int num_sms, cudaStream_t s) {
  if (q.n_obj == 0) return 0;
  uint64_t b = (q.n_obj + 255) / 256;
  if (b > uint64_t(num_sms) * 8) b = uint64_t(num_sms) * 8;
  frequency_reduce_kernel<<<(unsigned)b, 256, 0, s>>>(q);
  return 1;
}

}  // namespace drgpum
