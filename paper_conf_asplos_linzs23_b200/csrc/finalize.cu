// B4 tile_reduce_kernel + B5/B6 object_finalize_kernel (sm_100a).
//
// A6: per object, popcount of the bitmap (PAPER.md l.268
// "examines each data object's bitmap to compute the percentage of accessed
// elements"), lowest/highest accessed element, and the largest unaccessed
// chunk of Eq. (1) (l.191) -- an associative "bit-run" monoid combined over
// words, then over tiles, in order.  The hit-row scan walks the accessing APIs
// a_1 < ... < a_k of each object (Fig. 2's timestamp-augmented trace, l.232)
// and folds the temporary-idleness gaps (Def 3.6, l.164) and dead-write pairs
// (Def 3.7, l.168).
// A7: classification with the rules of l.244-249 and Def 3.8 / l.194, in
// exact integer arithmetic (readings R6-R12 of DESIGN.md).
#include "internal.cuh"
#include "../../include/drgpum.h"

namespace drgpum {

#define FULL_MASK 0xFFFFFFFFu
constexpr uint32_t kNoPos32 = 0xFFFFFFFFu;

// ---------------------------------------------------------------- bit runs
struct M32 { uint32_t len, pop, lo, hi, pre, suf, best; };

__device__ __forceinline__ M32 m32_identity() { return M32{0, 0, kNoPos32, kNoPos32, 0, 0, 0}; }

__device__ __forceinline__ M32 m32_word(uint32_t w, uint32_t nvalid) {
  if (nvalid == 0) return m32_identity();
  if (nvalid < 32) w &= (1u << nvalid) - 1u;
  M32 m;
  m.len = nvalid;
  if (w == 0) {
    m.pop = 0; m.lo = m.hi = kNoPos32; m.pre = m.suf = m.best = nvalid;
    return m;
  }
  m.pop = __popc(w);
  m.lo = __ffs(w) - 1;
  m.hi = 31 - __clz(w);
  m.pre = m.lo;
  m.suf = nvalid - 1 - m.hi;
  // zeros strictly between lo and hi: longest run of ones in y
  uint32_t y = ~w & ((1u << m.hi) - 1u) & ~((2u << m.lo) - 1u);
  uint32_t run = 0;
  while (y) { y &= y >> 1; ++run; }
  m.best = max(max(m.pre, m.suf), run);
  return m;
}

__device__ __forceinline__ M32 m32_cat(const M32& a, const M32& b) {
  M32 r;
  r.len = a.len + b.len;
  r.pop = a.pop + b.pop;
  r.lo = a.pop ? a.lo : (b.pop ? a.len + b.lo : kNoPos32);
  r.hi = b.pop ? a.len + b.hi : a.hi;
  r.pre = a.pop ? a.pre : a.len + b.pre;
  r.suf = b.pop ? b.suf : b.len + a.suf;
  r.best = max(max(a.best, b.best), a.suf + b.pre);
  return r;
}

__device__ __forceinline__ M32 m32_shfl_down(const M32& m, int d) {
  return M32{__shfl_down_sync(FULL_MASK, m.len, d), __shfl_down_sync(FULL_MASK, m.pop, d),
             __shfl_down_sync(FULL_MASK, m.lo, d), __shfl_down_sync(FULL_MASK, m.hi, d),
             __shfl_down_sync(FULL_MASK, m.pre, d), __shfl_down_sync(FULL_MASK, m.suf, d),
             __shfl_down_sync(FULL_MASK, m.best, d)};
}

__device__ __forceinline__ BitMonoid bm_identity() { return BitMonoid{0, 0, kNoPos, kNoPos, 0, 0, 0}; }

__device__ __forceinline__ BitMonoid bm_cat(const BitMonoid& a, const BitMonoid& b) {
  BitMonoid r;
  r.len = a.len + b.len;
  r.pop = a.pop + b.pop;
  r.lo = a.pop ? a.lo : (b.pop ? a.len + b.lo : kNoPos);
  r.hi = b.pop ? a.len + b.hi : a.hi;
  r.pre = a.pop ? a.pre : a.len + b.pre;
  r.suf = b.pop ? b.suf : b.len + a.suf;
  r.best = max(max(a.best, b.best), a.suf + b.pre);
  return r;
}

__device__ __forceinline__ BitMonoid bm_shfl_down(const BitMonoid& m, int d) {
  return BitMonoid{__shfl_down_sync(FULL_MASK, m.len, d), __shfl_down_sync(FULL_MASK, m.pop, d),
                   __shfl_down_sync(FULL_MASK, m.lo, d), __shfl_down_sync(FULL_MASK, m.hi, d),
                   __shfl_down_sync(FULL_MASK, m.pre, d), __shfl_down_sync(FULL_MASK, m.suf, d),
                   __shfl_down_sync(FULL_MASK, m.best, d)};
}

// B4: one warp per tile.  Each step covers 128 words (lane l: words 4l..4l+3
// via one 16-B load; object bitmaps and tiles start 4-word aligned).
__global__ void __launch_bounds__(256) tile_reduce_kernel(const uint32_t* __restrict__ orw,
    const Tile* __restrict__ tiles, uint64_t n_tiles, BitMonoid* __restrict__ out) {
  const int lane = threadIdx.x & 31;
  const uint64_t gwarp = (uint64_t(blockIdx.x) * blockDim.x + threadIdx.x) >> 5;
  const uint64_t nwarps = (uint64_t(gridDim.x) * blockDim.x) >> 5;
  for (uint64_t t = gwarp; t < n_tiles; t += nwarps) {
    const Tile tl = tiles[t];
    M32 acc = m32_identity();  // meaningful in lane 0
    for (uint32_t w0 = 0; w0 < tl.n_words; w0 += 128) {
      const uint32_t my = w0 + 4 * lane;
      uint4 v = make_uint4(0, 0, 0, 0);
      if (my < tl.n_words) v = *reinterpret_cast<const uint4*>(orw + tl.word_lo + my);
      // bits of this tile covered by word j: clamp(n_bits - 32*j, 0, 32)
      const uint64_t bit0 = uint64_t(my) * 32;
      const bool in = my < tl.n_words;
      const bool zero = (v.x | v.y | v.z | v.w) == 0;
      const bool ones = (v.x & v.y & v.z & v.w) == 0xFFFFFFFFu;
      const uint64_t chunk_bits = 128ull * 32;
      const bool full_chunk = uint64_t(w0) * 32 + chunk_bits <= tl.n_bits;
      M32 m;
      if (full_chunk && __all_sync(FULL_MASK, zero)) {
        m = M32{4096, 0, kNoPos32, kNoPos32, 4096, 4096, 4096};
        if (lane == 0) acc = m32_cat(acc, m);
        continue;
      }
      if (full_chunk && __all_sync(FULL_MASK, ones)) {
        m = M32{4096, 4096, 0, 4095, 0, 0, 0};
        if (lane == 0) acc = m32_cat(acc, m);
        continue;
      }
      auto nv = [&](uint64_t b) -> uint32_t {
        if (!in || b >= tl.n_bits) return 0;
        const uint64_t r = tl.n_bits - b;
        return r >= 32 ? 32u : uint32_t(r);
      };
      m = m32_word(v.x, nv(bit0));
      m = m32_cat(m, m32_word(v.y, nv(bit0 + 32)));
      m = m32_cat(m, m32_word(v.z, nv(bit0 + 64)));
      m = m32_cat(m, m32_word(v.w, nv(bit0 + 96)));
#pragma unroll
      for (int d = 1; d < 32; d <<= 1) {
        const M32 o = m32_shfl_down(m, d);
        m = m32_cat(m, o);
      }
      if (lane == 0) acc = m32_cat(acc, m);
    }
    if (lane == 0) {
      BitMonoid r;
      r.len = acc.len; r.pop = acc.pop;
      r.lo = acc.lo == kNoPos32 ? kNoPos : acc.lo;
      r.hi = acc.hi == kNoPos32 ? kNoPos : acc.hi;
      r.pre = acc.pre; r.suf = acc.suf; r.best = acc.best;
      out[t] = r;
    }
  }
}

// ---------------------------------------------------------------- hit rows
struct HitM {
  uint32_t cnt, first_ts, last_ts, fl;  // fl: bit0 first_w, bit1 first_cs, bit2 last_w, bit3 last_cs
  uint32_t ti_cnt, ti_max, dw;
  uint64_t ti_sum;
};

__device__ __forceinline__ HitM hit_identity() { return HitM{0, 0, 0, 0, 0, 0, 0, 0}; }

__device__ __forceinline__ HitM hit_cat(const HitM& a, const HitM& b, uint32_t x_ti) {
  if (a.cnt == 0) return b;
  if (b.cnt == 0) return a;
  HitM r;
  r.cnt = a.cnt + b.cnt;
  r.first_ts = a.first_ts;
  r.last_ts = b.last_ts;
  r.fl = (a.fl & 3u) | (b.fl & 12u);
  r.ti_cnt = a.ti_cnt + b.ti_cnt;
  r.ti_max = max(a.ti_max, b.ti_max);
  r.ti_sum = a.ti_sum + b.ti_sum;
  r.dw = a.dw + b.dw;
  const uint32_t gap = b.first_ts - a.last_ts - 1;   // APIs strictly between (R6)
  if (gap >= x_ti) { r.ti_cnt++; r.ti_max = max(r.ti_max, gap); r.ti_sum += gap; }
  // consecutive accessing APIs both memcpy/memset and both writing O (Def 3.7, R12)
  if ((a.fl & 4u) && (a.fl & 8u) && (b.fl & 1u) && (b.fl & 2u)) r.dw++;
  return r;
}

__device__ __forceinline__ HitM hit_shfl_down(const HitM& m, int d) {
  HitM r;
  r.cnt = __shfl_down_sync(FULL_MASK, m.cnt, d);
  r.first_ts = __shfl_down_sync(FULL_MASK, m.first_ts, d);
  r.last_ts = __shfl_down_sync(FULL_MASK, m.last_ts, d);
  r.fl = __shfl_down_sync(FULL_MASK, m.fl, d);
  r.ti_cnt = __shfl_down_sync(FULL_MASK, m.ti_cnt, d);
  r.ti_max = __shfl_down_sync(FULL_MASK, m.ti_max, d);
  r.dw = __shfl_down_sync(FULL_MASK, m.dw, d);
  r.ti_sum = __shfl_down_sync(FULL_MASK, m.ti_sum, d);
  return r;
}

// B5 + B6: one warp per object.
__global__ void __launch_bounds__(256) object_finalize_kernel(const FinalParams p) {
  const int lane = threadIdx.x & 31;
  const uint64_t gwarp = (uint64_t(blockIdx.x) * blockDim.x + threadIdx.x) >> 5;
  const uint64_t nwarps = (uint64_t(gridDim.x) * blockDim.x) >> 5;
  drgpum_object_stats_t* stats = static_cast<drgpum_object_stats_t*>(p.stats);
  drgpum_pattern_report_t* reps = static_cast<drgpum_pattern_report_t*>(p.reports);
  for (uint64_t o = gwarp; o < p.n_obj; o += nwarps) {
    // ---- bitmap tiles of o, in order
    const uint32_t t0 = p.tile_off[o], t1 = p.tile_off[o + 1];
    BitMonoid bm = bm_identity();
    for (uint32_t tb = t0; tb < t1; tb += 32) {
      BitMonoid m = (tb + lane < t1) ? p.tile_part[tb + lane] : bm_identity();
#pragma unroll
      for (int d = 1; d < 32; d <<= 1) m = bm_cat(m, bm_shfl_down(m, d));
      if (lane == 0) bm = bm_cat(bm, m);
    }
    // ---- hit row of o: 2 bits per access API inside its lifetime
    const DevObj ob = p.objs[o];
    const uint32_t nh = p.n_hit[o];
    const uint32_t nwords = (2 * nh + 31) / 32;
    HitM hm = hit_identity();
    for (uint32_t wb = 0; wb < nwords; wb += 32) {
      HitM m = hit_identity();
      const uint32_t wi = wb + lane;
      if (wi < nwords) {
        uint32_t w = p.orw[ob.hit_word + wi];
        while (w) {
          const uint32_t b = __ffs(w) - 1;
          const uint32_t j = b >> 1;                  // API slot inside this word
          const uint32_t pair = (w >> (2 * j)) & 3u;  // bit0 read, bit1 write
          w &= ~(3u << (2 * j));
          const uint32_t rank = ob.r_lo + wi * 16 + j;
          const uint32_t ts = __ldg(p.acc_ts + rank);
          const uint32_t cs = __ldg(p.acc_cs + rank);
          const uint32_t wr = (pair >> 1) & 1u;
          const HitM one{1, ts, ts, wr | (cs << 1) | (wr << 2) | (cs << 3), 0, 0, 0, 0};
          m = hit_cat(m, one, p.ti_min_idle);
        }
      }
#pragma unroll
      for (int d = 1; d < 32; d <<= 1) m = hit_cat(m, hit_shfl_down(m, d), p.ti_min_idle);
      if (lane == 0) hm = hit_cat(hm, m, p.ti_min_idle);
    }
    if (lane != 0) continue;
    // ---- stats (A6)
    const uint64_t n = (ob.end - ob.base) >> ob.shift;
    const uint32_t first = p.first[o], last = p.last[o];
    drgpum_object_stats_t st;
    st.n_elems = n;
    st.accessed = bm.pop;
    st.span_lo = bm.lo;   // kNoPos == UINT64_MAX
    st.span_hi = bm.hi;
    st.largest_unaccessed_run = bm.best;
    st.t_first = first;
    st.t_last = last;
    st.n_access_apis = hm.cnt;
    st._pad = 0;
    stats[o] = st;
    // cross-check of the two liveness folds (atomics vs hit rows), and of
    // bitmap vs hit row (an object with accessed elements has accessing APIs)
    const bool consistent = bm.len == n &&
        (hm.cnt ? (first == hm.first_ts && last == hm.last_ts && bm.pop > 0)
                : (first == kNever && last == 0 && bm.pop == 0));
    if (!consistent) atomicAdd(&p.ctr[C_CONSISTENCY], 1ull);
    // ---- patterns (A7)
    drgpum_pattern_report_t r;
    r.flags = 0; r.ea_distance = 0; r.ld_distance = 0; r.ti_ranges = 0;
    r.ti_max_idle = 0; r.dw_pairs = 0; r.ti_total_idle = 0;
    const bool used = hm.cnt > 0;
    const bool leak = ob.t_free == kNever;
    if (!used) r.flags |= DRGPUM_UA;
    if (leak) r.flags |= DRGPUM_ML;
    if (used) {
      if (hm.first_ts - ob.t_alloc >= 2) { r.flags |= DRGPUM_EA; r.ea_distance = hm.first_ts - ob.t_alloc; }
      if (!leak && ob.t_free - hm.last_ts >= 2) { r.flags |= DRGPUM_LD; r.ld_distance = ob.t_free - hm.last_ts; }
      r.ti_ranges = hm.ti_cnt; r.ti_max_idle = hm.ti_max; r.ti_total_idle = hm.ti_sum;
      r.dw_pairs = hm.dw;
      if (hm.ti_cnt) r.flags |= DRGPUM_TI;
      if (hm.dw) r.flags |= DRGPUM_DW;
    }
    using u128 = unsigned __int128;
    if (u128(bm.pop) * 100u < u128(p.oa_pct) * n) {
      r.flags |= DRGPUM_OA;
      const uint64_t unacc = n - bm.pop;
      if (unacc == 0 || u128(unacc - bm.best) * 100u < u128(p.frag_pct) * unacc)
        r.flags |= DRGPUM_OA_ACTIONABLE;
    }
    reps[o] = r;
  }
}

int launch_finalize(const FinalParams& p, int num_sms, cudaStream_t s) {
  if (p.n_obj == 0) return 0;
  const uint64_t tb = (p.n_tiles + 7) / 8;
  const unsigned g1 = (unsigned)(tb < uint64_t(num_sms) * 16 ? tb : uint64_t(num_sms) * 16);
  tile_reduce_kernel<<<g1 ? g1 : 1, 256, 0, s>>>(p.orw, p.tiles, p.n_tiles, p.tile_part);
  const uint64_t ob = (p.n_obj + 7) / 8;
  const unsigned g2 = (unsigned)(ob < uint64_t(num_sms) * 16 ? ob : uint64_t(num_sms) * 16);
  object_finalize_kernel<<<g2, 256, 0, s>>>(p);
  return 2;
}

// ---------------------------------------------------------------- utilities
__global__ void fill_u32_kernel(uint32_t* p, uint32_t v, uint64_t n) {
  for (uint64_t i = uint64_t(blockIdx.x) * blockDim.x + threadIdx.x; i < n;
       i += uint64_t(gridDim.x) * blockDim.x)
    p[i] = v;
}

int launch_fill_u32(uint32_t* p, uint32_t v, uint64_t n, cudaStream_t s) {
  if (!n) return 0;
  uint64_t b = (n + 255) / 256;
  if (b > 4096) b = 4096;
  fill_u32_kernel<<<(unsigned)b, 256, 0, s>>>(p, v, n);
  return 1;
}

// B7: OR n_src received slices into the owned words (after an all-to-all).
__global__ void __launch_bounds__(256) merge_or_kernel(uint32_t* __restrict__ dst,
    const uint32_t* __restrict__ src, uint32_t n_src, uint64_t stride, uint64_t n_words) {
  for (uint64_t i = uint64_t(blockIdx.x) * blockDim.x + threadIdx.x; i < n_words;
       i += uint64_t(gridDim.x) * blockDim.x) {
    uint32_t v = dst[i];
    for (uint32_t s = 0; s < n_src; ++s) v |= __ldg(src + s * stride + i);
    dst[i] = v;
  }
}

int launch_merge_or(uint32_t* dst, const uint32_t* src, uint32_t n_src, uint64_t src_stride,
                    uint64_t n_words, int num_sms, cudaStream_t s) {
  if (!n_words || !n_src) return 0;
  uint64_t b = (n_words + 255) / 256;
  if (b > uint64_t(num_sms) * 8) b = uint64_t(num_sms) * 8;
  merge_or_kernel<<<(unsigned)b, 256, 0, s>>>(dst, src, n_src, src_stride, n_words);
  return 1;
}

}  // namespace drgpum
