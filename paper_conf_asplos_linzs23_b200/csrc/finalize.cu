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
  // longest run of ones in y (y != ~0 here: it excludes bits lo and hi), by
  // binary lifting: A_j marks starts of runs >= 2^j (A_{j+1} = A_j & A_j >> 2^j);
  // cur marks starts of runs >= run; extend run by 2^j, j = 4..0, whenever a
  // run continues for another 2^j bits.  Branch-free, about 30 instructions.
  const uint32_t a1 = y & (y >> 1), a2 = a1 & (a1 >> 2), a3 = a2 & (a2 >> 4), a4 = a3 & (a3 >> 8);
  const uint32_t A[5] = {y, a1, a2, a3, a4};
  uint32_t cur = 0xFFFFFFFFu, run = 0;
#pragma unroll
  for (int j = 4; j >= 0; --j) {
    const uint32_t t = cur & (A[j] >> run);
    run += t ? (1u << j) : 0u;
    cur = t ? t : cur;
  }
  m.best = max(max(m.pre, m.suf), run);
  return m;
}

__device__ __forceinline__ M32 m32_cat(const M32& a, const M32& b) {
  M32 r;
  r.len = a.len + b.len;
  r.pop = a.pop + b.pop;
  r.lo = a.pop ? a.lo : (b.pop ? a.len + b.lo : kNoPos32);
  r.hi = b.pop ? a.len + b.hi : a.hi;
  r.pre = a.pre == a.len ? a.len + b.pre : a.pre;   // a has no 1 in the run view
  r.suf = b.suf == b.len ? b.len + a.suf : b.suf;
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
  r.pre = a.pre == a.len ? a.len + b.pre : a.pre;   // a has no 1 in the run view
  r.suf = b.suf == b.len ? b.len + a.suf : b.suf;
  r.best = max(max(a.best, b.best), a.suf + b.pre);
  return r;
}

__device__ __forceinline__ BitMonoid bm_shfl_down(const BitMonoid& m, int d) {
  return BitMonoid{__shfl_down_sync(FULL_MASK, m.len, d), __shfl_down_sync(FULL_MASK, m.pop, d),
                   __shfl_down_sync(FULL_MASK, m.lo, d), __shfl_down_sync(FULL_MASK, m.hi, d),
                   __shfl_down_sync(FULL_MASK, m.pre, d), __shfl_down_sync(FULL_MASK, m.suf, d),
                   __shfl_down_sync(FULL_MASK, m.best, d)};
}

// Longest run of zeros of u strictly between its lowest and highest set bit
// (0 with fewer than two set bits).  Binary lifting: A_j marks starts of runs
// >= 2^j (A_{j+1} = A_j & A_j >> 2^j); cur marks starts of runs >= run;
// extend run by 2^j, j = 4..0, whenever a run continues for another 2^j bits.
// Out of line: the second pass of tile_reduce_kernel is the only caller.
__device__ __noinline__ uint32_t interior_zero_run(uint32_t u) {
  if (u == 0) return 0;
  const uint32_t lo = __ffs(u) - 1, hi = 31 - __clz(u);
  if (hi <= lo + 1) return 0;
  const uint32_t y = ~u & ((1u << hi) - 1u) & ~((2u << lo) - 1u);
  const uint32_t a1 = y & (y >> 1), a2 = a1 & (a1 >> 2), a3 = a2 & (a2 >> 4), a4 = a3 & (a3 >> 8);
  const uint32_t A[5] = {y, a1, a2, a3, a4};
  uint32_t cur = 0xFFFFFFFFu, run = 0;
#pragma unroll
  for (int j = 4; j >= 0; --j) {
    const uint32_t t = cur & (A[j] >> run);
    run += t ? (1u << j) : 0u;
    cur = t ? t : cur;
  }
  return run;
}

// B4: one warp per tile (<= kTileWords = 1024 words of one object); lane l
// folds the 32 consecutive words [32l, 32l+32) sequentially (eight 16-B
// loads, the tile's lines shared through L1), then ONE warp join per tile:
// popcount by REDUX.SUM, lowest/highest accessed bit by ballot + one shuffle,
// and the longest zero run by joining every lane's leading zeros to the
// trailing zeros of the previous non-empty lane (ballot + one indexed shuffle
// + REDUX.MAX).  Bits past the object's last element are treated as 1
// ("sentinels") for the run view so no zero run extends past n_elems; they
// never count as accessed.  Zero runs inside one word (<= 30 bits) are skipped
// in the first pass and computed in a second pass only when the tile's other
// runs are all shorter than 30 -- otherwise they cannot change its longest
// run (dense strided sweeps need them; untouched or sparse regions do not).
// Blocks per SM (A/B on C2, tools/ab.sh): 4 (64 registers) 60.6 us of
// finalize; 5 (48, spills) 67.7; 6 (40, spills) 91.2.  Persistent variants
// with register prefetch (3 and 2 blocks/SM) 79.5 / 75.8, with a 3-stage
// cp.async ring (2 blocks/SM) 49.8 us of tile_reduce alone vs 40.8.
// r43 (ncu source page: 20.9M warp-instructions, stalls mostly long_sb on the
// tile loads): skipping pass-2 words equal to the last searched one or whose
// inner zeros cannot beat the running max 61.8 vs 60.5 us of finalize (not
// adopted); grid cap per SM (DRGPUM_TR_GRID_PER_SM) 4 / 8 / 16 / 64 blocks:
// 66.9 / 67.3 / 60.7 / 62.8 us of finalize -- 16 stays.
// Whole-tile closed form for all-ones / all-zeros tiles before the transpose
// (DRGPUM_TR_UNIFORM): 58.7 vs 60.7 us of finalize (3 rounds), adopted.
// DRGPUM_TR_UNIFORM=2 adds partial tiles (small objects, objects' last
// tiles) whose real bits are all 1 or all 0: C5 finalize 3.87 -> 2.72 ms,
// C2 unchanged (58.0 vs 58.3 us); adopted.
#ifndef DRGPUM_TR_BLOCKS
#define DRGPUM_TR_BLOCKS 4
#endif
#ifndef DRGPUM_TR_UNIFORM
#define DRGPUM_TR_UNIFORM 2
#endif
#ifndef DRGPUM_TR_SMALL
#define DRGPUM_TR_SMALL 1   // tiles of <= 128 words: 4 words per lane, no transpose
#endif
#ifndef DRGPUM_TR_GRID_PER_SM
#define DRGPUM_TR_GRID_PER_SM 16
#endif
// One tile of kLaneWords words per lane: 32 (full 1024-word tiles, lane l
// folds words [32l, 32l+32) after a transpose through buf) or 4 (tiles of at
// most 128 words -- small objects and objects' last tiles: the coalesced 16-B
// load already gives lane l words [4l, 4l+4), no transpose, 4-step folds).
// The run-view length of a 4-word-lane tile is 4096 bits; such tiles are
// always an object's last, so the length only has to cover its real bits.
template <uint32_t kLaneWords>
__device__ __forceinline__ void reduce_one_tile(uint32_t* __restrict__ orw, const Tile& tl, uint64_t t,
                                                BitMonoid* __restrict__ out, uint4* buf, int lane, bool consume) {
  constexpr uint32_t kLaneBits = kLaneWords * 32;
  static_assert(kLaneWords == 32 || kLaneWords == 4, "lane widths");
    const uint32_t nbits = uint32_t(tl.n_bits);
    const uint32_t w0 = kLaneWords * uint32_t(lane);
    uint4 v[kLaneWords / 4];
#pragma unroll
    for (int b = 0; b < int(kLaneWords / 4); ++b) {
      const uint32_t w = 128 * b + 4 * lane;
      const uint4* a = reinterpret_cast<const uint4*>(orw + tl.word_lo + w);
      v[b] = w < tl.n_words ? (consume ? *a : __ldg(a)) : make_uint4(0, 0, 0, 0);   // (no .nc path for words it rewrites)
    }
    if (consume) {   // reduce-and-clear: every word read is zeroed (the next reset skips the tiles)
#pragma unroll
      for (int b = 0; b < int(kLaneWords / 4); ++b) {
        const uint32_t w = 128 * b + 4 * lane;
        if (w < tl.n_words) *reinterpret_cast<uint4*>(orw + tl.word_lo + w) = make_uint4(0, 0, 0, 0);
      }
    }
#if DRGPUM_TR_UNIFORM
    // whole tiles that are all ones (dense sweeps) or all zeros (untouched
    // regions): AND / OR do not depend on word order, so they are decided on
    // the loaded vectors before the transpose and written in closed form
    if (nbits == 32u * kLaneBits) {
      uint32_t a = 0xFFFFFFFFu, o = 0u;
#pragma unroll
      for (int b = 0; b < int(kLaneWords / 4); ++b) {
        a &= v[b].x & v[b].y & v[b].z & v[b].w;
        o |= v[b].x | v[b].y | v[b].z | v[b].w;
      }
      const bool all1 = __all_sync(FULL_MASK, a == 0xFFFFFFFFu);
      const bool all0 = __all_sync(FULL_MASK, o == 0u);
      if (all1 || all0) {
        if (lane == 0) {
          const uint64_t L = 32u * kLaneBits;
          out[t] = all1 ? BitMonoid{L, L, 0, L - 1, 0, 0, 0} : BitMonoid{L, 0, kNoPos, kNoPos, L, L, L};
        }
        return;
      }
    }
#if DRGPUM_TR_UNIFORM > 1
    else {
      // a partial tile (an object's last, or a small object): every real bit
      // 1 (words past the end load as 0, the last word holds nbits % 32
      // valid bits) or every word 0; the run view then has the sentinels
      // [nbits, L) as ones.  Any stray bit past the end fails both checks.
      const uint32_t nw = tl.n_words;
      const uint32_t lastv = nbits - 32u * (nw - 1u);
      const uint32_t lastmask = lastv >= 32u ? 0xFFFFFFFFu : ((1u << lastv) - 1u);
      bool ones = true;
      uint32_t o = 0u;
#pragma unroll
      for (int b = 0; b < int(kLaneWords / 4); ++b) {
        const uint32_t w = 128u * b + 4u * lane;
        const uint32_t xs[4] = {v[b].x, v[b].y, v[b].z, v[b].w};
#pragma unroll
        for (int c = 0; c < 4; ++c) {
          const uint32_t wc = w + c;
          const uint32_t e = wc + 1u < nw ? 0xFFFFFFFFu : (wc + 1u == nw ? lastmask : 0u);
          ones = ones && xs[c] == e;
          o |= xs[c];
        }
      }
      const bool all1 = __all_sync(FULL_MASK, ones);
      const bool all0 = __all_sync(FULL_MASK, o == 0u);
      if (all1 || all0) {
        if (lane == 0) {
          const uint64_t L = 32u * kLaneBits;
          out[t] = all1 ? BitMonoid{L, nbits, 0, nbits - 1u, 0, 0, 0}
                        : BitMonoid{L, 0, kNoPos, kNoPos, nbits, 0, nbits};
        }
        return;
      }
    }
#endif
#endif
    if constexpr (kLaneWords == 32) {   // lane l <- words [32l, 32l+32) through the buffer
      __syncwarp();   // the previous tile's reads of buf are done
#pragma unroll
      for (int b = 0; b < int(kLaneWords / 4); ++b) {
        const uint32_t owner = 4 * b + (lane >> 3), chunk = lane & 7;
        buf[owner * 8 + (chunk ^ (owner & 7))] = v[b];
      }
      __syncwarp();
#pragma unroll
      for (int k = 0; k < int(kLaneWords / 4); ++k) v[k] = buf[lane * 8 + (k ^ (lane & 7))];
    }   // kLaneWords == 4: the coalesced load already gave lane l words [4l, 4l+4)
    // lane fold, branch-free per word: real popcount and the nonzero real
    // words (lowest / highest accessed bit at the end); run view: z = zeros
    // since the last 1, so a word with a 1 closes a zero run of z + ctz(u)
    // bits (the prefix run if it is the lane's first 1), then z = clz(u)
    uint32_t pop = 0, nzr = 0, z = 0, pre = kLaneBits, gapmax = 0;
    bool seen = false;
    auto step = [&](int j, uint32_t real, uint32_t u) {
      pop += __popc(real);
      nzr |= real ? (1u << j) : 0u;
      const bool has = u != 0u;
      const uint32_t c = z + __clz(__brev(u));
      gapmax = (has && seen) ? max(gapmax, c) : gapmax;
      pre = (has && !seen) ? c : pre;
      seen = seen || has;
      z = has ? __clz(u) : z + 32u;
    };
    // lane-uniform: does any of this lane's bits lie past the last element?
    const bool masked = (w0 + kLaneWords) * 32 > nbits;
    // all-ones / all-zeros lanes (dense sweeps, untouched regions) in closed
    // form: three-input ANDs / ORs over the 32 words instead of the fold
    uint32_t all_and = 0xFFFFFFFFu, all_or = 0u;
#pragma unroll
    for (int k = 0; k < int(kLaneWords / 4); ++k) {
      all_and &= v[k].x & v[k].y & v[k].z & v[k].w;
      all_or |= v[k].x | v[k].y | v[k].z | v[k].w;
    }
    const bool full = !masked && all_and == 0xFFFFFFFFu;
    const bool empty = !masked && all_or == 0u;
    auto views = [&](int j, uint32_t& real, uint32_t& run) {
      const uint4& q = v[j >> 2];
      const uint32_t x = (j & 3) == 0 ? q.x : (j & 3) == 1 ? q.y : (j & 3) == 2 ? q.z : q.w;
      const uint32_t bj = (w0 + j) * 32;
      const uint32_t nv = bj >= nbits ? 0u : min(32u, nbits - bj);
      const uint32_t vm = nv == 32 ? 0xFFFFFFFFu : ((1u << nv) - 1u);
      real = masked ? x & vm : x;
      run = masked ? real | ~vm : x;
    };
    if (full) {
      pop = kLaneBits; nzr = kLaneWords == 32 ? 0xFFFFFFFFu : (1u << kLaneWords) - 1u; z = 0; pre = 0; seen = true;
    } else if (empty) {
      z = kLaneBits;
    } else if (!masked) {
#pragma unroll
      for (int k = 0; k < int(kLaneWords / 4); ++k) {
        step(4 * k, v[k].x, v[k].x);
        step(4 * k + 1, v[k].y, v[k].y);
        step(4 * k + 2, v[k].z, v[k].z);
        step(4 * k + 3, v[k].w, v[k].w);
      }
    } else {
#pragma unroll
      for (int j = 0; j < int(kLaneWords); ++j) {
        uint32_t real, u;
        views(j, real, u);
        step(j, real, u);
      }
    }
    // lowest / highest accessed bit of the lane from its first / last nonzero
    // real word (read back from the transpose buffer, masked like above)
    uint32_t lo = kNoPos32, hi = kNoPos32;
    if (nzr) {
      const int jl = __ffs(nzr) - 1, jh = 31 - __clz(nzr);
      uint32_t xl, xh;
      if constexpr (kLaneWords == 32) {
        const uint32_t* wl = reinterpret_cast<const uint32_t*>(buf + lane * 8);
        xl = wl[4 * ((jl >> 2) ^ (lane & 7)) + (jl & 3)];
        xh = wl[4 * ((jh >> 2) ^ (lane & 7)) + (jh & 3)];
      } else {
        const uint32_t xs[4] = {v[0].x, v[0].y, v[0].z, v[0].w};
        xl = xs[jl & 3];
        xh = xs[jh & 3];
      }
      const uint32_t bl = (w0 + jl) * 32, bh = (w0 + jh) * 32;
      const uint32_t nl = min(32u, nbits - bl), nh = min(32u, nbits - bh);   // both words hold real bits
      const uint32_t ml = nl == 32 ? xl : xl & ((1u << nl) - 1u);
      const uint32_t mh = nh == 32 ? xh : xh & ((1u << nh) - 1u);
      lo = 32 * jl + __ffs(ml) - 1;
      hi = 32 * jh + 31 - __clz(mh);
    }
    const int first1 = seen ? int(pre) : -1;
    const int last1 = seen ? int(kLaneBits - 1 - z) : -1;
    M32 r;
    r.len = kLaneBits;
    r.pop = first1 >= 0 ? 1u : 0u;   // "has a 1 in the run view"
    r.pre = first1 >= 0 ? uint32_t(first1) : kLaneBits;
    r.suf = first1 >= 0 ? uint32_t(int(kLaneBits) - 1 - last1) : kLaneBits;
    r.best = first1 >= 0 ? max(gapmax, max(r.pre, r.suf)) : kLaneBits;
    // tile: combine the 32 lanes in order
    M32 acc;
    acc.len = 32 * kLaneBits;
    acc.pop = __reduce_add_sync(FULL_MASK, pop);
    const uint32_t nzp = __ballot_sync(FULL_MASK, pop != 0);
    if (nzp) {
      const int fl = __ffs(nzp) - 1, ll = 31 - __clz(nzp);
      acc.lo = kLaneBits * fl + __shfl_sync(FULL_MASK, lo, fl);
      acc.hi = kLaneBits * ll + __shfl_sync(FULL_MASK, hi, ll);
    } else {
      __shfl_sync(FULL_MASK, lo, 0);   // keep the shuffles convergent
      __shfl_sync(FULL_MASK, hi, 0);
      acc.lo = acc.hi = kNoPos32;
    }
    const uint32_t nz = __ballot_sync(FULL_MASK, r.pop != 0);   // lanes with a 1 in the run view
    const uint32_t below = nz & ((1u << lane) - 1u);
    const int i = below ? 31 - __clz(below) : -1;
    const uint32_t suf_i = __shfl_sync(FULL_MASK, r.suf, i < 0 ? 0 : i);
    const uint32_t run_j = (i < 0 ? 0u : suf_i + kLaneBits * uint32_t(lane - i - 1)) +
                           (i < 0 ? kLaneBits * lane : 0u) + r.pre;
    const uint32_t cand = r.pop ? max(r.best, run_j) : 0u;
    const uint32_t best = __reduce_max_sync(FULL_MASK, cand);
    if (nz == 0) {
      acc.pre = acc.suf = acc.best = 32 * kLaneBits;
      __shfl_sync(FULL_MASK, r.pre, 0);
      __shfl_sync(FULL_MASK, r.suf, 0);
    } else {
      const int f = __ffs(nz) - 1, l = 31 - __clz(nz);
      acc.pre = kLaneBits * f + __shfl_sync(FULL_MASK, r.pre, f);
      acc.suf = kLaneBits * (31 - l) + __shfl_sync(FULL_MASK, r.suf, l);
      acc.best = max(best, acc.suf);
    }
    // pass 2: zero runs inside single words (<= 30 bits) matter only if every
    // other run of the tile is shorter
    const bool mixed = !(full || empty);
    if (acc.best < 30 && __any_sync(FULL_MASK, mixed)) {
      uint32_t im = 0;
#pragma unroll
      for (int j = 0; j < int(kLaneWords); ++j) {
        if (!mixed) break;   // uniform lanes hold no word-interior zero run
        uint32_t real, u;
        views(j, real, u);
        if (u != 0u && u != 0xFFFFFFFFu) im = max(im, interior_zero_run(u));
      }
      acc.best = max(acc.best, __reduce_max_sync(FULL_MASK, im));
    }
    if (lane == 0) {
      BitMonoid r;
      r.len = acc.len;   // run-view length (sentinel bits only after an object's end)
      r.pop = acc.pop;
      r.lo = acc.lo == kNoPos32 ? kNoPos : acc.lo;
      r.hi = acc.hi == kNoPos32 ? kNoPos : acc.hi;
      r.pre = acc.pre; r.suf = acc.suf; r.best = acc.best;
      out[t] = r;
    }
}

#ifndef DRGPUM_FIN_UNTOUCHED
#define DRGPUM_FIN_UNTOUCHED 1   // tiles / hit rows of objects with first[o] = NEVER: closed forms, no loads
#endif
__global__ void __launch_bounds__(256, DRGPUM_TR_BLOCKS) tile_reduce_kernel(uint32_t* __restrict__ orw,
    const Tile* __restrict__ tiles, uint64_t n_tiles, BitMonoid* __restrict__ out, unsigned long long* ctr,
    const uint32_t* __restrict__ first, bool consume) {
  const int lane = threadIdx.x & 31;
  if (blockIdx.x == 0 && threadIdx.x == 0) ctr[C_CONSISTENCY] = 0;   // counted by object_finalize_kernel
  const uint64_t gwarp = (uint64_t(blockIdx.x) * blockDim.x + threadIdx.x) >> 5;
  const uint64_t nwarps = (uint64_t(gridDim.x) * blockDim.x) >> 5;
  static_assert(kTileWords == 1024, "transpose assumes 8 x 16-B chunks per lane");
  // per-warp 4-KB transpose buffer: the tile is read coalesced (lane l: words
  // 128b + 4l .. +3) and each 16-B chunk stored where its owning lane reads
  // it back; slot = owner * 8 + (chunk ^ (owner & 7)) keeps both sides free
  // of bank conflicts
  __shared__ uint4 s_tile[8][kTileWords / 4];
  uint4* buf = s_tile[threadIdx.x >> 5];
  for (uint64_t t = gwarp; t < n_tiles; t += nwarps) {
    const Tile tl = tiles[t];
    if (DRGPUM_FIN_UNTOUCHED && __ldg(first + tl.obj) == kNever) {
      // an object no record reached: its words are all zero (every
      // attributed record folds first[], the invariant the sparse reset uses
      // too) -- the all-zeros monoid of the tile's view, as the loads would give
      if (lane == 0) {
        const uint64_t L = (DRGPUM_TR_SMALL && tl.n_words <= 128) ? 4096u : 32768u, nb = tl.n_bits;
        out[t] = nb == L ? BitMonoid{L, 0, kNoPos, kNoPos, L, L, L} : BitMonoid{L, 0, kNoPos, kNoPos, nb, 0, nb};
      }
      continue;
    }
#if DRGPUM_TR_SMALL
    if (tl.n_words <= 128) { reduce_one_tile<4>(orw, tl, t, out, buf, lane, consume); continue; }
#endif
    reduce_one_tile<32>(orw, tl, t, out, buf, lane, consume);
  }
}

// B4b: one warp per group (<= 32 consecutive tiles of one object): ordered
// shuffle tree over the tile monoids.
template <bool kBatch>
__global__ void __launch_bounds__(256) group_reduce_kernel(const Group* __restrict__ groups,
    uint64_t n_groups, const BitMonoid* __restrict__ tile_part, BitMonoid* __restrict__ out) {
  const int lane = threadIdx.x & 31;
  const uint64_t gwarp = (uint64_t(blockIdx.x) * blockDim.x + threadIdx.x) >> 5;
  const uint64_t nwarps = (uint64_t(gridDim.x) * blockDim.x) >> 5;
  if (kBatch) {
  // 32 consecutive groups per warp: single-tile groups (small objects) are
  // copied lane-parallel, the others reduced one by one by the whole warp
  for (uint64_t g0 = gwarp * 32; g0 < n_groups; g0 += nwarps * 32) {
    const uint64_t g = g0 + lane;
    const Group gr = g < n_groups ? groups[g] : Group{0, 0};
    if (gr.n_tiles == 1) out[g] = tile_part[gr.tile_lo];
    uint32_t multi = __ballot_sync(FULL_MASK, gr.n_tiles > 1);
    while (multi) {
      const int j = __ffs(multi) - 1;
      multi &= multi - 1;
      const uint32_t tlo = __shfl_sync(FULL_MASK, gr.tile_lo, j), nt = __shfl_sync(FULL_MASK, gr.n_tiles, j);
      BitMonoid m = uint32_t(lane) < nt ? tile_part[tlo + lane] : bm_identity();
#pragma unroll
      for (int d = 1; d < 32; d <<= 1) m = bm_cat(m, bm_shfl_down(m, d));
      if (lane == 0) out[g0 + j] = m;
    }
  }
  return;
  }
  for (uint64_t g = gwarp; g < n_groups; g += nwarps) {
    const Group gr = groups[g];
    BitMonoid m = uint32_t(lane) < gr.n_tiles ? tile_part[gr.tile_lo + lane] : bm_identity();
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) m = bm_cat(m, bm_shfl_down(m, d));
    if (lane == 0) out[g] = m;
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
// acc_ts / acc_cs are staged in shared memory when they fit (the hit-row scan
// looks them up once per accessing API, on a dependent chain).
constexpr uint32_t kSmemAcc = 8192;

constexpr int kFinThreads = 256;


// A6 stats + A7 patterns of object o from its bitmap monoid and hit-row
// summary (one thread)
__device__ __forceinline__ void emit_object(const FinalParams& p, uint64_t o, const DevObj& ob,
                                            const BitMonoid& bm, const HitM& hm) {
  drgpum_object_stats_t* stats = static_cast<drgpum_object_stats_t*>(p.stats);
  drgpum_pattern_report_t* reps = static_cast<drgpum_pattern_report_t*>(p.reports);
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
  const bool consistent = bm.len >= n && (bm.pop == 0 || bm.hi < n) &&
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

// sequential fold of hit words [w_lo, w_hi) of an object (one lane)
struct HitFold {
  uint32_t cnt = 0, f_ts = 0, f_fl = 0, l_ts = 0, l_fl = 0, ti_cnt = 0, ti_max = 0, ti_sum = 0, dw = 0;
  __device__ __forceinline__ void add(uint32_t ts, uint32_t fl, uint32_t x_ti) {
    if (cnt == 0) {
      f_ts = ts; f_fl = fl;
    } else {
      const uint32_t gap = ts - l_ts - 1;               // APIs strictly between (R6)
      if (gap >= x_ti) { ++ti_cnt; ti_max = max(ti_max, gap); ti_sum += gap; }
      if (l_fl == 3u && fl == 3u) ++dw;                 // Def 3.7, R12
    }
    l_ts = ts; l_fl = fl; ++cnt;
  }
  template <typename TS, typename CS>
  __device__ __forceinline__ void words(const uint32_t* row, uint32_t w_lo, uint32_t w_hi, uint32_t r_lo,
                                        const TS& acc_ts, const CS& acc_cs, uint32_t x_ti) {
    constexpr uint32_t kB = 8;                          // words loaded per round trip
    for (uint32_t wb = w_lo; wb < w_hi; wb += kB) {
      uint32_t ws[kB];
#pragma unroll
      for (uint32_t j = 0; j < kB; ++j) ws[j] = wb + j < w_hi ? row[wb + j] : 0u;
      uint32_t any = 0;
#pragma unroll
      for (uint32_t j = 0; j < kB; ++j) any |= ws[j];
      if (!any) continue;                               // untouched stretch (unused objects: all of it)
#pragma unroll
      for (uint32_t j = 0; j < kB; ++j) {
      const uint32_t wi = wb + j;
      uint32_t w = ws[j];
      while (w) {
        const uint32_t j = uint32_t(__ffs(w) - 1) >> 1;    // API slot inside this word
        const uint32_t pair = (w >> (2 * j)) & 3u;         // bit0 read, bit1 write
        w &= ~(3u << (2 * j));
        const uint32_t rank = r_lo + wi * 16 + j;
        add(acc_ts[rank], (pair >> 1) | (uint32_t(acc_cs[rank]) << 1), x_ti);   // bit0 write, bit1 copy/set
      }
      }
    }
  }
};

template <bool kStaged, bool kLane>
__global__ void __launch_bounds__(kFinThreads) object_finalize_kernel(const FinalParams p) {
  extern __shared__ uint4 s_acc4[];     // [n_acc] ts (padded to 16 B), then [n_acc] cs bytes
  const uint32_t* acc_ts = p.acc_ts;
  const uint8_t* acc_cs = p.acc_cs;
  if (kStaged) {
    // 16-B copies (the workspace sections are 256-B aligned and padded, so
    // the rounded-up tails stay inside them); independent loads, one round trip
    const uint32_t nts = (p.n_acc + 3) / 4, ncs = (p.n_acc + 15) / 16;
    const uint4* g_ts = reinterpret_cast<const uint4*>(p.acc_ts);
    const uint4* g_cs = reinterpret_cast<const uint4*>(p.acc_cs);
    for (uint32_t i = threadIdx.x; i < nts + ncs; i += blockDim.x)
      s_acc4[i] = i < nts ? __ldg(g_ts + i) : __ldg(g_cs + (i - nts));
    __syncthreads();
    acc_ts = reinterpret_cast<const uint32_t*>(s_acc4);
    acc_cs = reinterpret_cast<const uint8_t*>(s_acc4 + nts);
  }
  const int lane = threadIdx.x & 31;
  const uint64_t gwarp = (uint64_t(blockIdx.x) * blockDim.x + threadIdx.x) >> 5;
  const uint64_t nwarps = (uint64_t(gridDim.x) * blockDim.x) >> 5;
  // 32 objects per warp step.  Small objects -- one bitmap group and a hit
  // row of at most kLaneHitWords words (C5's 10^6 objects) -- are finalized
  // by their own lane, 32 at once (their loads are independent, so the warp
  // overlaps 32 objects' latencies instead of walking them one by one); the
  // others one after the other by the whole warp.
  // kLane = false (mostly large objects, C2): one object per warp step.
  const uint32_t step = kLane ? 32u : 1u;
  for (uint64_t o0 = p.o_lo + gwarp * step; o0 < p.o_hi; o0 += nwarps * step) {
    const uint64_t ol = o0 + lane;
    bool small = false;
    if (kLane && ol < p.o_hi) {
      const uint32_t t0 = p.group_off[ol], t1 = p.group_off[ol + 1];
      const uint32_t nw = (2 * p.n_hit[ol] + 31) / 32;
      small = t1 - t0 <= 1 && nw <= kLaneHitWords;
      if (small) {
        const DevObj ob = p.objs[ol];
        const BitMonoid bm = t1 > t0 ? p.group_part[t0] : bm_identity();
        HitFold f;
        if (!DRGPUM_FIN_UNTOUCHED || p.first[ol] != kNever)   // untouched: an all-zero hit row
          f.words(p.orw + ob.hit_word, 0, nw, ob.r_lo, acc_ts, acc_cs, p.ti_min_idle);
        HitM hm = hit_identity();
        if (f.cnt) hm = HitM{f.cnt, f.f_ts, f.l_ts, 0, f.ti_cnt, f.ti_max, f.dw, f.ti_sum};
        emit_object(p, ol, ob, bm, hm);
      }
    }
    uint32_t big = kLane ? __ballot_sync(FULL_MASK, ol < p.o_hi && !small) : 1u;
    while (big) {
      const uint64_t o = o0 + uint32_t(__ffs(big) - 1);
      big &= big - 1;
      // ---- bitmap groups of o, in order
      const uint32_t t0 = p.group_off[o], t1 = p.group_off[o + 1];
      BitMonoid bm = bm_identity();
      if (t1 - t0 == 1) {
        bm = p.group_part[t0];
      } else {
        for (uint32_t tb = t0; tb < t1; tb += 32) {
          BitMonoid m = (tb + lane < t1) ? p.group_part[tb + lane] : bm_identity();
#pragma unroll
          for (int d = 1; d < 32; d <<= 1) m = bm_cat(m, bm_shfl_down(m, d));
          if (lane == 0) bm = bm_cat(bm, m);
        }
      }
      // ---- hit row of o: 2 bits per access API inside its lifetime.  Each
      // lane folds a contiguous run of hit words in order (count, first /
      // last accessing API with its write / copy-set flags, TI gaps and DW
      // pairs inside the run); the lanes are then joined at their
      // boundaries: the gap / pair between a lane's first API and the
      // previous non-empty lane's last one (one indexed shuffle), and warp
      // sums / maxima.
      const DevObj ob = p.objs[o];
      const uint32_t nwords = (DRGPUM_FIN_UNTOUCHED && p.first[o] == kNever) ? 0u : (2 * p.n_hit[o] + 31) / 32;
      const uint32_t per = (nwords + 31) / 32;
      const uint32_t wlo = min(nwords, lane * per), whi = min(nwords, wlo + per);
      HitFold f;
      f.words(p.orw + ob.hit_word, wlo, whi, ob.r_lo, acc_ts, acc_cs, p.ti_min_idle);
      const uint32_t nz = __ballot_sync(FULL_MASK, f.cnt != 0);
      HitM hm = hit_identity();
      if (nz) {
        const uint32_t below = nz & ((1u << lane) - 1u);
        const int pl = below ? 31 - __clz(below) : lane;
        const uint32_t p_ts = __shfl_sync(FULL_MASK, f.l_ts, pl);
        const uint32_t p_fl = __shfl_sync(FULL_MASK, f.l_fl, pl);
        uint32_t ti_cnt = f.ti_cnt, ti_max = f.ti_max, ti_sum = f.ti_sum, dw = f.dw;
        if (f.cnt && below) {
          const uint32_t gap = f.f_ts - p_ts - 1;
          if (gap >= p.ti_min_idle) { ++ti_cnt; ti_max = max(ti_max, gap); ti_sum += gap; }
          if (p_fl == 3u && f.f_fl == 3u) ++dw;
        }
        const int fl0 = __ffs(nz) - 1, fl1 = 31 - __clz(nz);
        hm.cnt = __reduce_add_sync(FULL_MASK, f.cnt);
        hm.first_ts = __shfl_sync(FULL_MASK, f.f_ts, fl0);
        hm.last_ts = __shfl_sync(FULL_MASK, f.l_ts, fl1);
        hm.ti_cnt = __reduce_add_sync(FULL_MASK, ti_cnt);
        hm.ti_max = __reduce_max_sync(FULL_MASK, ti_max);
        hm.ti_sum = __reduce_add_sync(FULL_MASK, ti_sum);   // sum of disjoint gaps < n_api < 2^31
        hm.dw = __reduce_add_sync(FULL_MASK, dw);
      }
      if (lane == 0) emit_object(p, o, ob, bm, hm);
    }
  }
}

int launch_finalize(const FinalParams& p, int num_sms, cudaStream_t s) {
  if (p.n_obj == 0) return 0;
  const uint64_t nt = p.t_hi - p.t_lo, ng = p.g_hi - p.g_lo, no = p.o_hi - p.o_lo;
  const uint64_t tb = (nt + 7) / 8;
  const uint64_t cap1 = uint64_t(num_sms) * DRGPUM_TR_GRID_PER_SM;
  const unsigned g1 = (unsigned)(tb < cap1 ? tb : cap1);
  if (p.skip_tiles) {   // consumed bitmaps: the monoids are in place; the consistency count restarts
    cudaMemsetAsync(p.ctr + C_CONSISTENCY, 0, sizeof(unsigned long long), s);
  } else {
  tile_reduce_kernel<<<g1 ? g1 : 1, 256, 0, s>>>(const_cast<uint32_t*>(p.orw), p.tiles + p.t_lo, nt,
                                                 p.tile_part + p.t_lo, p.ctr, p.first, p.consume);
  // mostly single-tile groups (many small objects, C5): 32 groups per warp,
  // single-tile ones copied lane-parallel (C5 finalize 2.77 -> 2.37 ms);
  // otherwise one warp per group (C2: the batched form 83 vs 58 us)
  const bool batch = nt < 2 * ng;
  const uint64_t gb = batch ? (ng + 255) / 256 : (ng + 7) / 8;
  const unsigned g3 = (unsigned)(gb < uint64_t(num_sms) * 16 ? gb : uint64_t(num_sms) * 16);
  if (batch)
    group_reduce_kernel<true><<<g3 ? g3 : 1, 256, 0, s>>>(p.groups + p.g_lo, ng, p.tile_part, p.group_part + p.g_lo);
  else
    group_reduce_kernel<false><<<g3 ? g3 : 1, 256, 0, s>>>(p.groups + p.g_lo, ng, p.tile_part, p.group_part + p.g_lo);
  }
  // lane-parallel small objects when they are the majority (host count,
  // FinalParams::n_small), else one object per warp
  // (only with enough objects to give every SM's warps 32 each: C5's 10^6;
  // C2 / C4 keep one object per warp, 7 / ~1500 us)
  const bool lane = 2 * p.n_small > no && no >= uint64_t(num_sms) * 32 * 32;
  const unsigned opb = lane ? kFinThreads : kFinThreads / 32;
  const uint64_t ob = (no + opb - 1) / opb;
  unsigned g2 = (unsigned)(ob < uint64_t(num_sms) * 16 ? ob : uint64_t(num_sms) * 16);
  if (g2 == 0) g2 = 1;
  const size_t sm = 16 * ((p.n_acc + 3) / 4 + (p.n_acc + 15) / 16);
  if (p.n_acc <= kSmemAcc) {
    if (lane) object_finalize_kernel<true, true><<<g2, kFinThreads, sm, s>>>(p);
    else object_finalize_kernel<true, false><<<g2, kFinThreads, sm, s>>>(p);
  } else {
    if (lane) object_finalize_kernel<false, true><<<g2, kFinThreads, 0, s>>>(p);
    else object_finalize_kernel<false, false><<<g2, kFinThreads, 0, s>>>(p);
  }
  return p.skip_tiles ? 1 : 3;
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

// Reset of a trace's dynamic state in one pass of 16-B stores: zeros, except
// the first[] section (16-B units [one_lo, one_hi)), which starts at NEVER.
__global__ void __launch_bounds__(256) reset_kernel(uint4* __restrict__ ws, uint64_t n16, uint64_t one_lo,
                                                   uint64_t one_hi) {
  const uint64_t stride = uint64_t(gridDim.x) * blockDim.x;
  for (uint64_t i = uint64_t(blockIdx.x) * blockDim.x + threadIdx.x; i < n16; i += stride) {
    const uint32_t v = (i >= one_lo && i < one_hi) ? 0xFFFFFFFFu : 0u;
    ws[i] = make_uint4(v, v, v, v);
  }
}

int launch_reset(void* ws, uint64_t bytes, uint64_t first_off, uint64_t first_bytes, int num_sms, cudaStream_t s) {
  const uint64_t n16 = (bytes + 15) / 16;
  if (!n16) return 0;
  uint64_t b = (n16 + 255) / 256;
  if (b > uint64_t(num_sms) * 16) b = uint64_t(num_sms) * 16;
  reset_kernel<<<(unsigned)b, 256, 0, s>>>(reinterpret_cast<uint4*>(ws), n16, first_off / 16,
                                            (first_off + first_bytes + 15) / 16);
  return 1;
}

// Sparse reset (drgpum_reset after the first bind): one warp per tile, then
// one warp per object for the hit rows; only objects with first[o] != NEVER
// hold nonzero words.  Tiles start 4-word aligned inside 4-word padded
// bitmaps, so whole 16-B stores cover them.
template <bool kLane>
__global__ void __launch_bounds__(256) reset_touched_kernel(uint32_t* __restrict__ orw,
    const Tile* __restrict__ tiles, uint64_t n_tiles, const DevObj* __restrict__ objs,
    const uint32_t* __restrict__ n_hit, const uint32_t* __restrict__ first, uint64_t n_obj) {
  const int lane = threadIdx.x & 31;
  const uint64_t gwarp = (uint64_t(blockIdx.x) * blockDim.x + threadIdx.x) >> 5;
  const uint64_t nwarps = (uint64_t(gridDim.x) * blockDim.x) >> 5;
  if (kLane) {
    // mostly small tiles (C5's 10^6 objects): 32 tiles per warp step, each
    // lane checks one and zeroes it itself if it is small; large touched
    // tiles are zeroed by the whole warp
    for (uint64_t t0 = gwarp * 32; t0 < n_tiles; t0 += nwarps * 32) {
      const uint64_t t = t0 + lane;
      bool big = false;
      if (t < n_tiles) {
        const Tile tl = tiles[t];
        if (__ldg(first + tl.obj) != kNever) {
          const uint32_t nv = (tl.n_words + 3) / 4;
          if (nv <= 32) {
            uint4* v = reinterpret_cast<uint4*>(orw + tl.word_lo);
            for (uint32_t i = 0; i < nv; ++i) v[i] = make_uint4(0, 0, 0, 0);
          } else {
            big = true;
          }
        }
      }
      uint32_t m = __ballot_sync(FULL_MASK, big);
      while (m) {
        const Tile tl = tiles[t0 + uint32_t(__ffs(m) - 1)];
        m &= m - 1;
        uint4* v = reinterpret_cast<uint4*>(orw + tl.word_lo);
        const uint32_t nv = (tl.n_words + 3) / 4;
        for (uint32_t i = lane; i < nv; i += 32) v[i] = make_uint4(0, 0, 0, 0);
      }
    }
  } else {
    // one warp per tile (the zeroing is the work: up to 1024 words each)
    for (uint64_t t = gwarp; t < n_tiles; t += nwarps) {
      const Tile tl = tiles[t];
      if (__ldg(first + tl.obj) == kNever) continue;   // warp-uniform
      uint4* v = reinterpret_cast<uint4*>(orw + tl.word_lo);
      const uint32_t nv = (tl.n_words + 3) / 4;
      for (uint32_t i = lane; i < nv; i += 32) v[i] = make_uint4(0, 0, 0, 0);
    }
  }
  for (uint64_t o0 = gwarp * 32; o0 < n_obj; o0 += nwarps * 32) {   // hit rows, 32 objects per step
    const uint64_t o = o0 + lane;
    const bool touched = o < n_obj && __ldg(first + o) != kNever;
    uint64_t hw = 0;
    uint32_t nw = 0;
    if (touched) {
      hw = objs[o].hit_word;
      nw = (2 * n_hit[o] + 31) / 32;
    }
    uint32_t m = __ballot_sync(FULL_MASK, touched);
    while (m) {
      const int j = __ffs(m) - 1;
      m &= m - 1;
      const uint64_t h = __shfl_sync(FULL_MASK, hw, j);
      const uint32_t n = __shfl_sync(FULL_MASK, nw, j);
      for (uint32_t i = lane; i < n; i += 32) orw[h + i] = 0;
    }
  }
}

int launch_reset_touched(uint32_t* orw, const Tile* tiles, uint64_t n_tiles, const DevObj* objs,
                         const uint32_t* n_hit, const uint32_t* first, uint64_t n_obj, bool lane_tiles,
                         int num_sms, cudaStream_t s) {
  const uint64_t work = n_tiles > n_obj / 32 ? n_tiles : n_obj / 32;
  if (!n_tiles && !n_obj) return 0;
  uint64_t b = (work + 7) / 8 + 1;
  if (b > uint64_t(num_sms) * 16) b = uint64_t(num_sms) * 16;
  if (lane_tiles)
    reset_touched_kernel<true><<<(unsigned)b, 256, 0, s>>>(orw, tiles, n_tiles, objs, n_hit, first, n_obj);
  else
    reset_touched_kernel<false><<<(unsigned)b, 256, 0, s>>>(orw, tiles, n_tiles, objs, n_hit, first, n_obj);
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

// B7' (peer memory): the one exchange step as ONE kernel per rank over
// NVLink peer pointers (symmetric memory / CUDA IPC).  Rank r owns the word
// slice [w_lo, w_hi) of the OR words and the object slice [o_lo, o_hi): it
// reads its slice from every peer's shadow (its own included), ORs /
// MINs / MAXes them, and stores the result into every peer's slice, so that
// after a barrier every rank holds the merged shadow.  Slices of different
// ranks are disjoint, so the ranks' kernels never touch the same word.  Rank
// 0 also sums the counters.  OR / MIN / MAX / SUM are associative and
// commutative: the result is bit-exact for any number of ranks.
__global__ void __launch_bounds__(256) merge_peers_kernel(const MergePeersParams q) {
  const uint64_t tid = uint64_t(blockIdx.x) * blockDim.x + threadIdx.x;
  const uint64_t nth = uint64_t(gridDim.x) * blockDim.x;
  // OR words, 16 B at a time (the slice bounds are multiples of 4 words)
  const uint64_t v_lo = q.w_lo / 4, v_hi = q.w_hi / 4;
  for (uint64_t i = v_lo + tid; i < v_hi; i += nth) {
    uint4 v = make_uint4(0, 0, 0, 0);
    for (uint32_t r = 0; r < q.n_peers; ++r) {
      const uint4 x = __ldcg(reinterpret_cast<const uint4*>(q.peer[r] + q.or_off) + i);
      v.x |= x.x; v.y |= x.y; v.z |= x.z; v.w |= x.w;
    }
    for (uint32_t r = 0; r < q.n_peers; ++r)
      __stcg(reinterpret_cast<uint4*>(q.peer[r] + q.or_off) + i, v);
  }
  for (uint64_t o = q.o_lo + tid; o < q.o_hi; o += nth) {
    uint32_t f = 0xFFFFFFFFu, l = 0;
    for (uint32_t r = 0; r < q.n_peers; ++r) {
      f = min(f, __ldcg(reinterpret_cast<const uint32_t*>(q.peer[r] + q.first_off) + o));
      l = max(l, __ldcg(reinterpret_cast<const uint32_t*>(q.peer[r] + q.last_off) + o));
    }
    for (uint32_t r = 0; r < q.n_peers; ++r) {
      __stcg(reinterpret_cast<uint32_t*>(q.peer[r] + q.first_off) + o, f);
      __stcg(reinterpret_cast<uint32_t*>(q.peer[r] + q.last_off) + o, l);
    }
  }
  if (q.rank == 0 && tid < 5) {   // records, attributed, unattributed, clipped, invalid
    unsigned long long sum = 0;
    for (uint32_t r = 0; r < q.n_peers; ++r)
      sum += __ldcg(reinterpret_cast<const unsigned long long*>(q.peer[r] + q.ctr_off) + tid);
    for (uint32_t r = 0; r < q.n_peers; ++r)
      __stcg(reinterpret_cast<unsigned long long*>(q.peer[r] + q.ctr_off) + tid, sum);
  }
}

int launch_merge_peers(const MergePeersParams& q, int num_sms, cudaStream_t s) {
  const uint64_t work = max((q.w_hi - q.w_lo) / 4, q.o_hi - q.o_lo);
  uint64_t b = (work + 255) / 256;
  if (b > uint64_t(num_sms) * 8) b = uint64_t(num_sms) * 8;
  if (b < 1) b = 1;
  merge_peers_kernel<<<(unsigned)b, 256, 0, s>>>(q);
  return 1;
}

// B7'': owned merge.  Reads rank r's objects' shadow from every peer and
// stores the OR / MIN / MAX into rank r's workspace only (no write-back to
// the peers: each rank finalizes its own objects, gather_peers shares the
// results).  NVLink traffic per rank: (P-1)/P of the shadow read, nothing
// written remotely -- half of merge_peers_kernel's.
__global__ void __launch_bounds__(256) merge_owned_kernel(const MergeOwnedParams q) {
  const uint64_t tid = uint64_t(blockIdx.x) * blockDim.x + threadIdx.x;
  const uint64_t nth = uint64_t(gridDim.x) * blockDim.x;
  uint8_t* const own = q.peer[q.rank];
  for (uint64_t i = q.b_lo / 4 + tid; i < q.b_hi / 4; i += nth) {   // bitmaps: 4-word aligned per object
    uint4 v = make_uint4(0, 0, 0, 0);
    for (uint32_t r = 0; r < q.n_peers; ++r) {
      const uint4 x = __ldcg(reinterpret_cast<const uint4*>(q.peer[r] + q.or_off) + i);
      v.x |= x.x; v.y |= x.y; v.z |= x.z; v.w |= x.w;
    }
    __stcg(reinterpret_cast<uint4*>(own + q.or_off) + i, v);
  }
  for (uint64_t w = q.h_lo + tid; w < q.h_hi; w += nth) {           // hit rows
    uint32_t v = 0;
    for (uint32_t r = 0; r < q.n_peers; ++r) v |= __ldcg(reinterpret_cast<const uint32_t*>(q.peer[r] + q.or_off) + w);
    __stcg(reinterpret_cast<uint32_t*>(own + q.or_off) + w, v);
  }
  for (uint64_t o = q.o_lo + tid; o < q.o_hi; o += nth) {
    uint32_t f = 0xFFFFFFFFu, l = 0;
    for (uint32_t r = 0; r < q.n_peers; ++r) {
      f = min(f, __ldcg(reinterpret_cast<const uint32_t*>(q.peer[r] + q.first_off) + o));
      l = max(l, __ldcg(reinterpret_cast<const uint32_t*>(q.peer[r] + q.last_off) + o));
    }
    __stcg(reinterpret_cast<uint32_t*>(own + q.first_off) + o, f);
    __stcg(reinterpret_cast<uint32_t*>(own + q.last_off) + o, l);
  }
  if (q.rank == 0 && tid < 5) {   // records, attributed, unattributed, clipped, invalid
    unsigned long long sum = 0;
    for (uint32_t r = 0; r < q.n_peers; ++r)
      sum += __ldcg(reinterpret_cast<const unsigned long long*>(q.peer[r] + q.ctr_off) + tid);
    for (uint32_t r = 0; r < q.n_peers; ++r)
      __stcg(reinterpret_cast<unsigned long long*>(q.peer[r] + q.ctr_off) + tid, sum);
  }
}

int launch_merge_owned(const MergeOwnedParams& q, int num_sms, cudaStream_t s) {
  const uint64_t work = max(max((q.b_hi - q.b_lo) / 4, q.h_hi - q.h_lo), max(q.o_hi - q.o_lo, uint64_t(5)));
  uint64_t b = (work + 255) / 256;
  if (b > uint64_t(num_sms) * 8) b = uint64_t(num_sms) * 8;
  merge_owned_kernel<<<(unsigned)b, 256, 0, s>>>(q);
  return 1;
}

// NVLS (NVLink SHARP): one load through the multicast mapping returns the OR
// of every rank's copy, reduced in the NVSwitch.
__device__ __forceinline__ uint64_t mc_or64(const void* a) {
  uint64_t v;
  asm volatile("multimem.ld_reduce.relaxed.sys.global.or.b64 %0, [%1];" : "=l"(v) : "l"(a) : "memory");
  return v;
}
__device__ __forceinline__ uint32_t mc_or32(const void* a) {
  uint32_t v;
  asm volatile("multimem.ld_reduce.relaxed.sys.global.or.b32 %0, [%1];" : "=r"(v) : "l"(a) : "memory");
  return v;
}

// B7'' sparse: the owned merge reading only what a peer wrote.  A peer's
// words of object o are nonzero only if its first[o] is set (every bit is
// attributed or merged together with a first-use fold), so kernel 1 (one
// warp per owned object) reads every peer's first/last, folds MIN / MAX,
// records the mask of peers that touched o, and ORs those peers' hit rows;
// kernel 2 (one warp per owned tile) ORs the bitmap tiles of the peers in the
// mask.  Objects touched only here keep their local words (no traffic);
// objects no rank touched cost two u32 reads per peer.  With record-range
// shards most objects live inside one shard's time window, so the NVLink
// traffic drops from (P-1)/P of the shadow to about the touched part of it.
__global__ void __launch_bounds__(256) merge_owned_objects_kernel(const MergeOwnedParams q) {
  const int lane = threadIdx.x & 31;
  const uint64_t gwarp = (uint64_t(blockIdx.x) * blockDim.x + threadIdx.x) >> 5;
  const uint64_t nwarps = (uint64_t(gridDim.x) * blockDim.x) >> 5;
  uint8_t* const own = q.peer[q.rank];
  for (uint64_t o = q.o_lo + gwarp; o < q.o_hi; o += nwarps) {
    uint32_t f = 0xFFFFFFFFu, l = 0;
    unsigned long long mask = 0;
    for (uint32_t p0 = 0; p0 < q.n_peers; p0 += 32) {
      const uint32_t p = p0 + lane;
      uint32_t fp = 0xFFFFFFFFu, lp = 0;
      if (p < q.n_peers) {
        fp = __ldcg(reinterpret_cast<const uint32_t*>(q.peer[p] + q.first_off) + o);
        lp = __ldcg(reinterpret_cast<const uint32_t*>(q.peer[p] + q.last_off) + o);
      }
      f = min(f, __reduce_min_sync(FULL_MASK, fp));
      l = max(l, __reduce_max_sync(FULL_MASK, lp));
      mask |= (unsigned long long)__ballot_sync(FULL_MASK, fp != 0xFFFFFFFFu) << p0;
    }
    if (lane == 0) {
      reinterpret_cast<uint32_t*>(own + q.first_off)[o] = f;
      reinterpret_cast<uint32_t*>(own + q.last_off)[o] = l;
      q.pmask[o] = mask;
    }
    if ((mask & ~(1ull << q.rank)) == 0) continue;   // nobody else touched o
    const uint64_t hw = q.objs[o].hit_word;
    const uint32_t nw = (2 * q.n_hit[o] + 31) / 32;
    const bool nvls = q.mc && __popcll(mask & ~(1ull << q.rank)) >= 2;   // the switch ORs the copies
    for (uint32_t i = lane; i < nw; i += 32) {
      uint32_t v = 0;
      if (nvls) {
        v = mc_or32(q.mc + q.or_off + 4 * (hw + i));
      } else {
        for (unsigned long long m = mask; m; m &= m - 1)
          v |= __ldcg(reinterpret_cast<const uint32_t*>(q.peer[__ffsll(m) - 1] + q.or_off) + hw + i);
      }
      reinterpret_cast<uint32_t*>(own + q.or_off)[hw + i] = v;
    }
  }
  const uint64_t tid = uint64_t(blockIdx.x) * blockDim.x + threadIdx.x;
  if (q.rank == 0 && tid < 5) {   // records, attributed, unattributed, clipped, invalid
    unsigned long long sum = 0;
    for (uint32_t r = 0; r < q.n_peers; ++r)
      sum += __ldcg(reinterpret_cast<const unsigned long long*>(q.peer[r] + q.ctr_off) + tid);
    for (uint32_t r = 0; r < q.n_peers; ++r)
      __stcg(reinterpret_cast<unsigned long long*>(q.peer[r] + q.ctr_off) + tid, sum);
  }
}

__global__ void __launch_bounds__(256) merge_owned_tiles_kernel(const MergeOwnedParams q) {
  const int lane = threadIdx.x & 31;
  const uint64_t gwarp = (uint64_t(blockIdx.x) * blockDim.x + threadIdx.x) >> 5;
  const uint64_t nwarps = (uint64_t(gridDim.x) * blockDim.x) >> 5;
  uint8_t* const own = q.peer[q.rank];
  for (uint64_t t = q.t_lo + gwarp; t < q.t_hi; t += nwarps) {
    const Tile tl = q.tiles[t];
    const unsigned long long mask = q.pmask[tl.obj];
    if ((mask & ~(1ull << q.rank)) == 0) continue;   // warp-uniform: local words are final
    const uint32_t nv = (tl.n_words + 3) / 4;
    if (q.mc && __popcll(mask & ~(1ull << q.rank)) >= 2) {   // NVLS: one reduced load per 8 B
      const uint8_t* mp = q.mc + q.or_off + 4 * tl.word_lo;
      for (uint32_t i = lane; i < nv; i += 32) {
        const uint64_t a = mc_or64(mp + 16 * i), b = mc_or64(mp + 16 * i + 8);
        reinterpret_cast<uint4*>(own + q.or_off + 4 * tl.word_lo)[i] =
            make_uint4(uint32_t(a), uint32_t(a >> 32), uint32_t(b), uint32_t(b >> 32));
      }
      continue;
    }
    for (uint32_t i = lane; i < nv; i += 32) {
      uint4 v = make_uint4(0, 0, 0, 0);
      for (unsigned long long m = mask; m; m &= m - 1) {
        const uint4 x = __ldcg(reinterpret_cast<const uint4*>(q.peer[__ffsll(m) - 1] + q.or_off + 4 * tl.word_lo) + i);
        v.x |= x.x; v.y |= x.y; v.z |= x.z; v.w |= x.w;
      }
      reinterpret_cast<uint4*>(own + q.or_off + 4 * tl.word_lo)[i] = v;
    }
  }
}

int launch_merge_owned_sparse(const MergeOwnedParams& q, int num_sms, cudaStream_t s) {
  const uint64_t no = q.o_hi - q.o_lo, nt = q.t_hi - q.t_lo;
  uint64_t b1 = (max(no, uint64_t(1)) + 7) / 8;
  if (b1 > uint64_t(num_sms) * 16) b1 = uint64_t(num_sms) * 16;
  merge_owned_objects_kernel<<<(unsigned)b1, 256, 0, s>>>(q);
  if (!nt) return 1;
  uint64_t b2 = (nt + 7) / 8;
  if (b2 > uint64_t(num_sms) * 16) b2 = uint64_t(num_sms) * 16;
  merge_owned_tiles_kernel<<<(unsigned)b2, 256, 0, s>>>(q);
  return 2;
}

// B7'': gather of the finalized stats / reports of rank r's objects into
// every peer (u32 copies; both sections are 4-B multiples per object).
__global__ void __launch_bounds__(256) gather_peers_kernel(const GatherParams q) {
  const uint64_t tid = uint64_t(blockIdx.x) * blockDim.x + threadIdx.x;
  const uint64_t nth = uint64_t(gridDim.x) * blockDim.x;
  const uint8_t* const own = q.peer[q.rank];
  for (uint32_t r = 0; r < q.n_peers; ++r) {
    if (r == q.rank) continue;
    for (uint64_t i = q.s_lo / 4 + tid; i < q.s_hi / 4; i += nth)
      reinterpret_cast<uint32_t*>(q.peer[r] + q.stats_off)[i] =
          reinterpret_cast<const uint32_t*>(own + q.stats_off)[i];
    for (uint64_t i = q.r_lo / 4 + tid; i < q.r_hi / 4; i += nth)
      reinterpret_cast<uint32_t*>(q.peer[r] + q.reports_off)[i] =
          reinterpret_cast<const uint32_t*>(own + q.reports_off)[i];
  }
  if (tid == 0) {
    const unsigned long long mine = reinterpret_cast<const unsigned long long*>(own + q.ctr_off)[C_CONSISTENCY];
    for (uint32_t r = 0; r < q.n_peers; ++r)
      reinterpret_cast<unsigned long long*>(q.peer[r] + q.cons_off)[q.rank] = mine;
  }
}

int launch_gather_peers(const GatherParams& q, int num_sms, cudaStream_t s) {
  const uint64_t work = max((q.s_hi - q.s_lo) / 4, (q.r_hi - q.r_lo) / 4);
  uint64_t b = (work + 255) / 256;
  if (b > uint64_t(num_sms) * 4) b = uint64_t(num_sms) * 4;
  if (b < 1) b = 1;
  gather_peers_kernel<<<(unsigned)b, 256, 0, s>>>(q);
  return 1;
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
