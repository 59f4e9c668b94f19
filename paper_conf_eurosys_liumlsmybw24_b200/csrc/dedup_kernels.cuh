// dedup_kernels.cuh — configuration dedup on the device:
// a streaming 64-bit hash of every candidate of a tiled batch, and an open-addressing
// visited set in HBM with deterministic first-occurrence semantics across calls.
// The hash and the table entry layout are specified in include/aceso.h.
#pragma once
#include <cstdint>

namespace aceso {

constexpr uint64_t kHashSeed = 0x243F6A8885A308D3ull;
constexpr uint64_t kHashPos = 0x9E3779B97F4A7C15ull;

__device__ __forceinline__ uint64_t hash_mix(uint64_t x) {  // splitmix64 finalizer
  x ^= x >> 30;
  x *= 0xBF58476D1CE4E5B9ull;
  x ^= x >> 27;
  x *= 0x94D049BB133111EBull;
  return x ^ (x >> 31);
}
// contribution of word i (position-tagged)
__device__ __forceinline__ uint64_t hash_word(uint64_t w, uint32_t i) {
  return hash_mix(w ^ ((uint64_t)(i + 1) * kHashPos));
}

// CTA = 4 warps = one tile of 32 candidates; warp w hashes the chunks k = w (mod 4) of the
// tile (each chunk read is 512 contiguous bytes: coalesced, every byte read once) with all
// of its loads in flight; the word contributions are summed (the hash is a sum of
// position-tagged mixes), partial sums meet in shared memory.
constexpr int kHashWarps = 4;
constexpr int kHashMaxLoads = 8;  // chunks per warp per round (registers: 8 x uint4)

__global__ void __launch_bounds__(kHashWarps * 32) hash_kernel(const uint4 *__restrict__ codes,
                                                              const uint64_t *__restrict__ hdr,
                                                              int64_t n, int32_t L,
                                                              uint64_t *__restrict__ out) {
  __shared__ uint64_t part[kHashWarps][32];
  const int32_t nch = (L + 15) / 16;
  const int32_t lf = L & ~7;  // bytes in full code words
  const int32_t r = L & 7;
  const uint32_t lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const int64_t n_tiles = (n + 31) / 32;
  for (int64_t tile = blockIdx.x; tile < n_tiles; tile += gridDim.x) {
    const int64_t c = tile * 32 + lane;
    const bool act = c < n;
    const uint4 *src = codes + (size_t)tile * nch * 32 + lane;
    const uint64_t hd = act ? __ldcs(hdr + c) : 0ull;
    uint64_t h = 0;
    for (int32_t k0 = warp; k0 < nch; k0 += kHashWarps * kHashMaxLoads) {
      uint4 v[kHashMaxLoads];
#pragma unroll
      for (int u = 0; u < kHashMaxLoads; ++u) {
        const int32_t k = k0 + u * kHashWarps;
        v[u] = (act && k < nch) ? __ldcs(src + (size_t)k * 32) : make_uint4(0, 0, 0, 0);
      }
#pragma unroll
      for (int u = 0; u < kHashMaxLoads; ++u) {
        const int32_t k = k0 + u * kHashWarps;
        if (k >= nch) break;
        const uint64_t w0 = ((uint64_t)v[u].y << 32) | v[u].x, w1 = ((uint64_t)v[u].w << 32) | v[u].z;
        const int32_t b0 = 16 * k, b1 = 16 * k + 8;
        if (b0 + 8 <= lf) h += hash_word(w0, 2 * k);
        if (b1 + 8 <= lf) h += hash_word(w1, 2 * k + 1);
        // the word holding the last L % 8 code bytes also takes the header's low bytes
        const uint64_t keep = (1ull << (8 * r)) - 1ull;
        const uint32_t nw = (uint32_t)(lf / 8);
        if (r != 0 && b0 == lf) {
          h += hash_word((w0 & keep) | (hd << (8 * r)), nw);
          h += hash_word(hd >> (64 - 8 * r), nw + 1);
        }
        if (r != 0 && b1 == lf) {
          h += hash_word((w1 & keep) | (hd << (8 * r)), nw);
          h += hash_word(hd >> (64 - 8 * r), nw + 1);
        }
      }
    }
    part[warp][lane] = h;
    __syncthreads();
    if (warp == 0) {
      h = part[0][lane] + part[1][lane] + part[2][lane] + part[3][lane];
      if (r == 0) h += hash_word(hd, (uint32_t)(lf / 8));  // the header is a word of its own
      h = hash_mix(kHashSeed + h);
      if (h == 0) h = 1;
      if (act) __stcs(out + c, h);
    }
    __syncthreads();
  }
}

struct VisitedEntry {
  unsigned long long hash;  // 0 = empty
  unsigned long long tag;   // max of ~(epoch << 40 | index) over the inserts
};

__device__ __forceinline__ uint64_t visit_tag(uint32_t epoch, int64_t i) {
  return ~(((uint64_t)epoch << 40) | (uint64_t)i);
}

// pass 1: insert every hash and max-reduce the (complemented) first-occurrence tag
__global__ void __launch_bounds__(256) visit_insert_kernel(const uint64_t *__restrict__ hs, int64_t n,
                                                           uint32_t epoch, VisitedEntry *table,
                                                           uint64_t mask, uint32_t *status) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n;
       i += (int64_t)gridDim.x * blockDim.x) {
    const unsigned long long h = hs[i];
    uint64_t slot = h & mask;
    for (uint64_t probe = 0;; ++probe) {
      if (probe > mask) {  // every slot holds another hash: full
        atomicExch(status, 1u);
        break;
      }
      const unsigned long long prev = atomicCAS(&table[slot].hash, 0ull, h);
      if (prev == 0ull || prev == h) {
        atomicMax(&table[slot].tag, (unsigned long long)visit_tag(epoch, i));
        break;
      }
      slot = (slot + 1) & mask;
    }
  }
}

// pass 2: a candidate is a duplicate unless it is the entry's first occurrence
__global__ void __launch_bounds__(256) visit_flag_kernel(const uint64_t *__restrict__ hs, int64_t n,
                                                         uint32_t epoch, const VisitedEntry *table,
                                                         uint64_t mask, uint8_t *__restrict__ dup) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n;
       i += (int64_t)gridDim.x * blockDim.x) {
    const uint64_t h = hs[i];
    uint64_t slot = h & mask;
    uint8_t d = 1;
    for (uint64_t probe = 0; probe <= mask; ++probe) {
      const uint64_t e = table[slot].hash;
      if (e == h) {
        d = table[slot].tag == visit_tag(epoch, i) ? 0 : 1;
        break;
      }
      if (e == 0) break;  // not inserted (table was full): status already set
      slot = (slot + 1) & mask;
    }
    dup[i] = d;
  }
}

}  // namespace aceso
