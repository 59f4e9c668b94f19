// enum_kernel.cuh — exhaustive enumeration of stage partitions on the device (SURVEY §8(f)
// NEXT(4), the Exp#4 mathematical-programming baseline): candidate r of a
// (p, code, header) family puts stage heads at op 0 and at the cut positions of the r-th
// (p-1)-subset of {1, ..., L-1} in colex order; every op carries `code` (tp, dp, recompute
// bits). Written straight into the tiled layout aceso_eval streams.
#pragma once
#include <cstdint>

namespace aceso {

// C(n, k) for k <= 7, saturated at 2^63 (only compared against ranks < 2^62); each step
// C(n-k+t-1, t-1) * (n-k+t) / t is exact in 128 bits
__host__ __device__ __forceinline__ uint64_t binom_sat(uint64_t n, uint32_t k) {
  if (n < k) return 0;
  unsigned __int128 v = 1;
  for (uint32_t t = 1; t <= k; ++t) {
    v = v * (n - k + t) / t;
    if (v >= ((unsigned __int128)1 << 63)) return 1ull << 63;
  }
  return (uint64_t)v;
}

// Thread = candidate (lane = slot in its tile: coalesced 16-byte stores of whole chunks).
__global__ void __launch_bounds__(256) enum_cuts_kernel(int32_t L, uint32_t k /* p - 1 */, uint32_t code,
                                                        uint64_t hdr, int64_t first, int64_t n,
                                                        uint4 *__restrict__ tiled, uint64_t *__restrict__ hout) {
  const int32_t nch = (L + 15) / 16;
  const uint32_t fill = (code & 0xfeu) * 0x01010101u;  // no head bits
  for (int64_t c = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; c < n; c += (int64_t)gridDim.x * blockDim.x) {
    // colex unranking: cut_i = 1 + largest x with C(x, i) <= r, i = k .. 1
    uint64_t r = (uint64_t)(first + c);
    uint32_t cut[8];
    uint32_t hi = (uint32_t)L - 1u;  // x in [i - 1, hi)
    for (uint32_t i = k; i >= 1; --i) {
      uint32_t lo = i - 1u, h = hi;  // C(lo, i) = 0 <= r; find the largest x < h with C(x, i) <= r
      while (h - lo > 1u) {
        const uint32_t mid = (lo + h) >> 1;
        if (binom_sat(mid, i) <= r) lo = mid; else h = mid;
      }
      r -= binom_sat(lo, i);
      cut[i] = lo + 1u;
      hi = lo;
    }
    const int64_t tile = c >> 5;
    const uint32_t lane = (uint32_t)(c & 31);
    uint32_t ci = 1;  // next cut (ascending: cut[1] < cut[2] < ...)
    for (int32_t ch = 0; ch < nch; ++ch) {
      uint32_t w[4] = {fill, fill, fill, fill};
      if (ch == 0) w[0] |= 1u;  // op 0 opens stage 0
      while (ci <= k && cut[ci] < (uint32_t)(16 * ch + 16)) {
        const uint32_t o = cut[ci] - 16u * (uint32_t)ch;
        w[o >> 2] |= 1u << (8u * (o & 3u));
        ++ci;
      }
      const int32_t pad = 16 * ch + 16 - L;  // bytes >= L are zero
      if (pad > 0) {
#pragma unroll
        for (int q = 0; q < 4; ++q) {
          const int32_t v = 16 - pad - 4 * q;  // valid bytes of word q
          w[q] = v >= 4 ? w[q] : v <= 0 ? 0u : (w[q] & ((1u << (8 * v)) - 1u));
        }
      }
      tiled[((size_t)tile * nch + ch) * 32 + lane] = make_uint4(w[0], w[1], w[2], w[3]);
    }
    hout[c] = hdr;
  }
}

}  // namespace aceso
