// Device-side expansion of a program's bursts into 16-byte access records
// (SURVEY.md §8(d) "B9").  Input generation only: this file holds none of
// the method's arithmetic (no lookup, no bitmap, no liveness) and is shared
// by nothing under oracle/ or the product library.  It computes exactly the
// pure function tracegen/records.py:gen_records computes on the host --
//   AFFINE : elem_j = start + (j*stride) mod span
//   RANDOM : elem_j = start + splitmix64(seed ^ (b << 32) ^ j) mod span
//   RANGE  : elem_j = start            (stride 0, span 1)
//   RAW    : addr = base
//   addr = base + elem_j * E, size = access_size, meta = ts | is_write << 31
// in the same wrapping u64 arithmetic -- so that C3-C5 traces larger than
// host memory can be generated chunk by chunk on the GPU.  Bit-identity with
// the host generator is a GPU test (tests/test_gpu_tracegen.py).
#include <cstdint>
#include <cuda_runtime.h>

namespace {

struct Burst {   // tracegen/layout.py BURST_DTYPE (64 B)
  uint64_t base, start, stride, span, count;
  uint32_t ts, elem, access_size, obj;
  uint8_t pattern, is_write, pad[6];
};
static_assert(sizeof(Burst) == 64, "BURST_DTYPE layout");
struct Rec { uint64_t addr; uint32_t size, meta; };

constexpr uint8_t kRandom = 1, kRaw = 3;   // AFFINE (0) and RANGE (2) need no special case

__device__ __forceinline__ uint64_t splitmix64(uint64_t x) {
  uint64_t z = x + 0x9E3779B97F4A7C15ull;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}

// last b with prefix[b] <= i
__device__ __forceinline__ uint64_t find_burst(const uint64_t* prefix, uint64_t nb, uint64_t i) {
  uint64_t lo = 0, hi = nb;   // prefix[0] = 0 <= i < prefix[nb]
  while (hi - lo > 1) {
    const uint64_t mid = (lo + hi) >> 1;
    if (prefix[mid] <= i) lo = mid; else hi = mid;
  }
  return lo;
}

// one warp per run of 1024 consecutive records; lane l writes records
// i0 + 32k + l (coalesced 16-B stores)
__global__ void __launch_bounds__(256) gen_kernel(const Burst* __restrict__ bursts,
    const uint64_t* __restrict__ prefix, uint64_t nb, uint64_t seed, uint64_t i0, uint64_t i1,
    Rec* __restrict__ out) {
  const int lane = threadIdx.x & 31;
  const uint64_t gwarp = (uint64_t(blockIdx.x) * blockDim.x + threadIdx.x) >> 5;
  const uint64_t nwarps = (uint64_t(gridDim.x) * blockDim.x) >> 5;
  constexpr uint64_t kRun = 1024;
  for (uint64_t r0 = i0 + gwarp * kRun; r0 < i1; r0 += nwarps * kRun) {
    uint64_t b = find_burst(prefix, nb, r0 + lane < i1 ? r0 + lane : r0);
    for (uint64_t i = r0 + lane; i < r0 + kRun && i < i1; i += 32) {
      while (prefix[b + 1] <= i) ++b;
      const Burst& B = bursts[b];
      const uint64_t j = i - prefix[b];
      const uint64_t span = B.span ? B.span : 1;
      uint64_t elem = B.start + (j * B.stride) % span;
      if (B.pattern == kRandom) elem = B.start + splitmix64(seed ^ (b << 32) ^ j) % span;
      uint64_t addr = B.base + elem * uint64_t(B.elem);
      if (B.pattern == kRaw) addr = B.base;
      out[i - i0] = Rec{addr, B.access_size, B.ts | (uint32_t(B.is_write) << 31)};
    }
  }
}

}  // namespace

extern "C" {

// Records [i0, i1) of the program (bursts[nb], prefix[nb + 1], both device
// pointers) into out[0, i1 - i0) (device, 16-B aligned), stream-ordered.
// Returns 0, or the cudaError_t of the launch.
__attribute__((visibility("default"))) int tg_gen_records(const void* bursts, const uint64_t* prefix,
    uint64_t nb, uint64_t seed, uint64_t i0, uint64_t i1, void* out, void* stream) {
  if (i1 <= i0) return 0;
  const uint64_t runs = (i1 - i0 + 1023) / 1024;
  uint64_t blocks = (runs + 7) / 8;
  if (blocks > 148 * 16) blocks = 148 * 16;
  gen_kernel<<<unsigned(blocks), 256, 0, static_cast<cudaStream_t>(stream)>>>(
      static_cast<const Burst*>(bursts), prefix, nb, seed, i0, i1, static_cast<Rec*>(out));
  return int(cudaGetLastError());
}

}
