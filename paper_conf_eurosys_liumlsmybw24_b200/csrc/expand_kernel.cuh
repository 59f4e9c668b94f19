// expand_kernel.cuh — on-device candidate generation (Table 1,
// P:L163-176): candidate = base encoding + up to 6 byte-range patches (include/aceso.h,
// aceso_cand), expanded straight into the tiled layout the eval kernels stream.
#pragma once
#include <cstdint>

#include "../../include/aceso.h"

namespace aceso {

// mask of the bytes [lo, hi) of a 4-byte word (lo, hi relative to the word, clamped)
__device__ __forceinline__ uint32_t byte_range_mask(int lo, int hi) {
  lo = max(lo, 0);
  hi = min(hi, 4);
  if (hi <= lo) return 0u;
  const uint32_t mh = hi >= 4 ? 0xffffffffu : ((1u << (8 * hi)) - 1u);
  const uint32_t ml = (1u << (8 * lo)) - 1u;  // lo <= 3
  return mh & ~ml;
}

// The 16 codes of chunk k (ops 16k..16k+15) of a candidate: its base's bytes with the
// patches applied in order (include/aceso.h, ACESO_PATCH_*).
__device__ __forceinline__ uint4 patched_chunk(const uint4 *__restrict__ brow, const uint16_t *__restrict__ ranks,
                                               uint32_t base, int32_t stride, int32_t L, const aceso_cand &cd,
                                               int np, int32_t k) {
  const uint4 v = __ldg(brow + k);
  uint32_t w[4] = {v.x, v.y, v.z, v.w};
  const int32_t c0 = 16 * k;
  for (int i = 0; i < np; ++i) {
    const aceso_patch pt = cd.patch[i];
    const int32_t a = min((int32_t)pt.a, L), b = min((int32_t)pt.b, L);
    if (b <= c0 || a >= c0 + 16 || b <= a) continue;
    if (a <= c0 && b >= c0 + 16 && pt.kind != ACESO_PATCH_RANK_RC) {  // the whole chunk
      if (pt.kind == ACESO_PATCH_MASK) {
        const uint32_t m0 = pt.v0 * 0x01010101u, m1 = pt.v1 * 0x01010101u;
#pragma unroll
        for (int q = 0; q < 4; ++q) w[q] = (w[q] & m0) | m1;
      } else if (pt.kind == ACESO_PATCH_ADD) {
        const uint32_t d = (uint32_t)(uint8_t)(((int8_t)pt.v0 << 1) + ((int8_t)pt.v1 << 5)) * 0x01010101u;
#pragma unroll
        for (int q = 0; q < 4; ++q) w[q] = __vadd4(w[q], d);
      }
      continue;
    }
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      const int32_t o = c0 + 4 * q;
      const uint32_t m = byte_range_mask(a - o, b - o);
      if (m == 0u) continue;
      uint32_t nv = w[q];
      if (pt.kind == ACESO_PATCH_MASK) {
        nv = (w[q] & (pt.v0 * 0x01010101u)) | (pt.v1 * 0x01010101u);
      } else if (pt.kind == ACESO_PATCH_ADD) {
        const uint32_t d = (uint32_t)(uint8_t)(((int8_t)pt.v0 << 1) + ((int8_t)pt.v1 << 5));
        nv = __vadd4(w[q], d * 0x01010101u);  // per-byte add; the fields stay in range
      } else if (pt.kind == ACESO_PATCH_RANK_RC && ranks != nullptr) {
        const uint32_t kk = (uint32_t)pt.v0 | ((uint32_t)pt.v1 << 8);
        const uint16_t *rk = ranks + ((size_t)base * 2 + (pt.v2 & 1u)) * stride + o;
#pragma unroll
        for (int t = 0; t < 4; ++t) {
          if (!((m >> (8 * t)) & 0xffu)) continue;
          if ((uint32_t)__ldg(rk + t) < kk) {
            if (pt.v2 & 2u) nv &= ~(0x10u << (8 * t));
            else nv |= 0x10u << (8 * t);
          }
        }
      }
      w[q] = (w[q] & ~m) | (nv & m);
    }
  }
  return make_uint4(w[0], w[1], w[2], w[3]);
}

// Thread = candidate (lane = its slot in the tile, so every 16-byte store of a warp
// fills one contiguous 512-byte chunk of the tiled output).
__global__ void __launch_bounds__(256) expand_kernel(const uint8_t *__restrict__ bases,
                                                     const uint16_t *__restrict__ ranks, int32_t nb,
                                                     int32_t L, const aceso_cand *__restrict__ cands,
                                                     int64_t n, uint4 *__restrict__ tiled,
                                                     uint64_t *__restrict__ hdr) {
  const int32_t nch = (L + 15) / 16;
  const int32_t stride = nch * 16;
  for (int64_t c = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; c - (threadIdx.x & 31) < n;
       c += (int64_t)gridDim.x * blockDim.x) {
    if (c >= n) continue;
    const aceso_cand cd = cands[c];
    const uint32_t base = min(cd.base, (uint32_t)nb - 1u);
    const uint4 *brow = reinterpret_cast<const uint4 *>(bases + (size_t)base * stride);
    const int np = min((int)cd.n_patch, 6);
    const int64_t tile = c >> 5;
    const uint32_t lane = (uint32_t)(c & 31);
    for (int32_t k = 0; k < nch; ++k) {
      const uint4 w = patched_chunk(brow, ranks, base, stride, L, cd, np, k);
      tiled[((size_t)tile * nch + k) * 32 + lane] = w;
    }
    hdr[c] = (uint64_t)cd.mbs_log2 | ((uint64_t)cd.p << 8);
  }
}

}  // namespace aceso
