// aux_kernels.cuh — argmin over a written summary (aceso_select) and the
// row-major -> tiled repack (aceso_pack_rowmajor). sm_100a.
#pragma once
#include "common.cuh"

namespace aceso {

// Selection over SoA summaries (Alg. 1 GetBestOf; "better").
__global__ void __launch_bounds__(256) select_kernel(const uint64_t *__restrict__ iter,
                                                     const uint64_t *__restrict__ mem,
                                                     const uint32_t *__restrict__ info, int64_t n,
                                                     int64_t gofs, unsigned char *sel,
                                                     int64_t n_total, uint32_t ib) {
  __shared__ uint64_t s_ck[8];
  __shared__ int64_t s_idx[8];
  uint64_t best = ~0ull;
  int64_t bidx = INT64_MAX;
  for (int64_t c = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; c < n;
       c += (int64_t)gridDim.x * blockDim.x) {
    const uint32_t f = info[c];
    if (f & ACESO_INFO_INVALID) continue;
    const uint64_t ck = (f & ACESO_INFO_OOM) ? ((1ull << 62) | mem[c]) : iter[c];
    if (key_less(ck, gofs + c, best, bidx)) {
      best = ck;
      bidx = gofs + c;
    }
  }
  block_select_finish(best, bidx, sel, n_total, ib, s_ck, s_idx);
}

// Row-major [n][L] -> tiled (32 candidates x 16 ops per 512-byte chunk). One
// thread writes one lane's 16 bytes of one chunk.
__global__ void __launch_bounds__(256) pack_kernel(const uint8_t *__restrict__ src, int64_t n,
                                                   int32_t L, uint4 *__restrict__ dst,
                                                   int64_t total_vec) {
  const int nch = (L + 15) / 16;
  for (int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v < total_vec;
       v += (int64_t)gridDim.x * blockDim.x) {
    const int64_t lane = v & 31;
    const int64_t rest = v >> 5;
    const int64_t ch = rest % nch;
    const int64_t tile = rest / nch;
    const int64_t c = tile * 32 + lane;
    uint32_t w[4] = {0u, 0u, 0u, 0u};
    if (c < n) {
      const uint8_t *row = src + c * (int64_t)L;
#pragma unroll
      for (int k = 0; k < 16; ++k) {
        const int64_t j = ch * 16 + k;
        const uint32_t b = j < L ? (uint32_t)row[j] : 0u;
        w[k >> 2] |= b << (8 * (k & 3));
      }
    }
    dst[v] = make_uint4(w[0], w[1], w[2], w[3]);
  }
}

// row-major dimension bytes [n][L] -> tiled plane: one u16 per (candidate, 16-op chunk)
__global__ void __launch_bounds__(256) pack_dims_kernel(const uint8_t *__restrict__ src, int64_t n, int L,
                                                        uint16_t *__restrict__ dst, int64_t total) {
  const int nch = (L + 15) / 16;
  for (int64_t u = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; u < total; u += (int64_t)gridDim.x * blockDim.x) {
    // u enumerates the plane: ((tile * nch + k) * 32 + lane)
    const int64_t lane = u & 31, tk = u >> 5;
    const int64_t tile = tk / nch, k = tk % nch;
    const int64_t c = tile * 32 + lane;
    uint32_t v = 0;
    if (c < n)
      for (int i = 0; i < 16; ++i) {
        const int64_t j = k * 16 + i;
        if (j < L && src[c * L + j]) v |= 1u << i;
      }
    dst[u] = (uint16_t)v;
  }
}

}  // namespace aceso
