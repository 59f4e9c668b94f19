// common.cuh — shared device-side definitions of libaceso (sm_100a).
//
// Packed profile tables (built on the host by aceso_load_profile from the
// int64 op-cost database of §3.3) and the kernel parameter block.
// DESIGN.md §5 documents the layout; the encoding is the one of include/aceso.h.
#pragma once
#include <cstdint>

#include "../../include/aceso.h"

namespace aceso {

constexpr int kWarps = 8;                    // warps per CTA in the eval kernel
constexpr int kThreads = kWarps * 32;
constexpr int kMaxOps = 16384;               // ops per model (per-op type offsets staged in smem)
constexpr uint32_t kTypeStride = 32;         // bytes per op type in every smem table

// Hot table R[b][tpl][type][rc] : 16-byte record (u32 each)
//   x = S'  = fwd_comp + fwd_comm + bwd_comp + bwd_comm + rc*(fwd_comp + fwd_comm)   (R7)
//   y = A   = rc ? keep : act                                                          (R3)
//   z = e   = peak + rc*(act - keep)                                                   (R3, R4)
//   w = W   = param+grad bytes + optimizer bytes at this tp
// Memory fields (y, z, w) are stored in units of 2^mem_shift bytes, where mem_shift is
// the largest power of two dividing every memory value of the profile (<= 2^16), so
// the sums stay exact: Mem_i = (Wst + infl * A + E) << mem_shift.
// DP table D[tpl][type][dpl] : u32 DP gradient all-reduce ns, 8 dpl slots per 32-byte entry
// Type table T[j] : u16 type_j for every op (16-entry chunks, zero padded)
// Quad tables (4 consecutive ops j = 4q..4q+3 with the same run and rc; sums exact in u32):
//   QO[q]            : {sig * RUNS * 32, sig * n_tp * 32} or {kNone, 0} (no quad sums)
//   QT[sig][run][rc] : 16 B {sum S', sum A, max e, sum W} over the quad's 4 op types
//   QD[sig][tpl][dpl]: u32 sum of DP all-reduce ns (8 dpl slots)
//   QF[sig][run][rc] : u32 sum of comp (FULL only)
// Full table F[b][tpl][type][rc] : u32 comp = fwd_comp + bwd_comp + rc*fwd_comp (8 B per type)
// Cold table K[b][tpl][type] : 16 bytes {reshard, p2p_fwd, p2p_bwd, 0}  (R5, R13), read
//   from global memory (L1/L2) at events only — after the shared blob in the same allocation
struct Tables {
  uint32_t offR, offD, offT, offQO, offQT, offQD;  // byte offsets in the staged blob (smem)
  uint32_t offF, offQF;                            // FULL-only tables (staged after bytes)
  uint32_t bytes;                   // bytes staged to shared memory (multiple of 16)
  uint32_t bytes_full;              // bytes staged including the F table
  uint32_t offK;                    // byte offset of the cold table in the global blob
  uint32_t bytesK;                  // bytes of the cold table
  uint32_t k_smem;                  // 1: the cold table is staged to shared memory too
  // dense-kernel tables (dense_kernel.cuh): the same records TYPE-major, so that the lanes of
  // a warp (same op, same type, different runs) read neighbouring records, not one bank
  //   DR[type][run][rc] 16 B, DD[type][tpl][dpl] u32 (8 slots), DK[type][run] 16 B,
  //   DT[j] u16, DF[type][run][rc] u32 (FULL) — at dOff in the blob, offsets relative to it
  uint32_t dOff, dR, dD, dK, dT, dF, dbytes, dbytes_full;
};

struct EvalParams {
  const uint4 *codes;     // tiled op codes
  const uint64_t *hdr;    // [n] headers
  int64_t n;              // candidates in this call
  int64_t gofs;           // global index of candidate 0
  int64_t n_tiles;
  int32_t L, nch, T, n_tp, n_dp, n_b, G;
  uint64_t Bg, C;
  uint32_t mem_shift;     // memory fields are stored >> mem_shift (exact)
  const uint4 *blob;      // packed tables (global)
  Tables tab;
  // outputs
  uint64_t *iter_ns, *max_mem;
  uint32_t *info;
  uint64_t *stage_T, *stage_mem, *stage_comp, *stage_comm;
  int32_t p_max;
  // selection
  unsigned char *sel;     // aceso_select_result + counter + per-CTA partials
  int64_t n_total;
  uint32_t ib;            // index bits of the packed key
  // event kernel (event_kernel.cuh): position-prefix tables in global memory, see EvTables
  const uint4 *px;        // [RUNS][L+1] x 2: {PS, PA} {PW, PC}   (u64 prefix sums, rc = 0)
  const uint4 *kx;        // [RUNS][L+1]    : {reshard_j, p2p_bwd_j, p2p_fwd_{j-1}, 0}
  const uint64_t *pd;     // [n_tp * n_dp][L+1] DP all-reduce prefix sums
  const uint32_t *st;     // [levels][RUNS][L] sparse table of e0 = peak (range max)
  const uint4 *qr;        // [nsig][RUNS][16] x 2: {dS, dA} {E1, 0, dC} rc deltas of a quad pattern
  const uint4 *qr8;       // [nsig8][RUNS][256] x 2: the same per octet pattern (8-chunk slots)
  const uint32_t *qo8;    // [2 * nch] octet signature offsets (sig8 * RUNS * 256)
  uint32_t runs;          // RUNS = n_b * n_tp
  uint32_t qo_bytes;      // bytes of the per-quad signature table staged to shared memory
  uint32_t qo_off;        // its byte offset in the event blob
  const unsigned char *evblob;
  // scan kernel (scan_kernel.cuh), exact u64 tables in global memory:
  const uint4 *sx;        // [RUNS][L+1] x 2: {PS, PA} {PW, PC}  u64 prefix sums at rc = 0
  const uint4 *sk;        // [RUNS][L+1]    : {reshard_j, p2p_bwd_j, p2p_fwd_{j-1}, 0} (u32 ns)
  const uint64_t *sd;     // [n_tp * n_dp][L+1] DP all-reduce prefix sums
  const void *ss;         // [levels][RUNS][L] range-max table of peak >> es (u32, or u64 when wide)
  const uint4 *sq;        // [nsig][RUNS][16] x 2: {dS, dA} {e1 >> es, dC} u64 recompute deltas
  const uint32_t *sqo;    // [4 * nch] per-quad signature record offset (staged to shared memory)
  uint32_t qo_words;
  uint32_t es;            // transient-memory values are stored in units of 2^es bytes
  uint32_t tw_q, tw_r;    // scan kernel: tiles per warp (quotient / remainder over all warps)
  uint32_t sc_resolve;    // scan kernel: resolve recompute-only chunks in the compacted pass
  const unsigned char *dims;  // dense kernel with DIMS: tiled dimension plane (aceso_eval_dims)
  uint32_t n_minus;       // Eq. 2 steady-phase microbatches N - n_minus: 1 (reading R1), 0 (ACESO_PIPE_LITERAL)
  unsigned long long *gkey;  // aceso_eval_global: the job's global key (local or peer-mapped), or null
};

// select buffer layout: [0,32) result, [32,40) completion counter, [64, ...) partials (16 B each)
constexpr int kSelCounterOff = 32;
constexpr int kSelPartialOff = 64;

__device__ __forceinline__ bool key_less(uint64_t a, int64_t ai, uint64_t b, int64_t bi) {
  return a < b || (a == b && ai < bi);
}

// lexicographic argmin of (ck, idx) across the warp; result valid in every lane
__device__ __forceinline__ void warp_argmin(uint64_t &ck, int64_t &idx) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    uint64_t ock = __shfl_xor_sync(0xffffffffu, ck, o);
    int64_t oidx = __shfl_xor_sync(0xffffffffu, idx, o);
    if (key_less(ock, oidx, ck, idx)) {
      ck = ock;
      idx = oidx;
    }
  }
}

// Block-level argmin + grid-level completion (last CTA reduces all partials and
// writes the final result). Called by every thread of the CTA.
__device__ __forceinline__ void block_select_finish(uint64_t ck, int64_t idx, unsigned char *sel,
                                                    int64_t n_total, uint32_t ib,
                                                    uint64_t *s_ck, int64_t *s_idx,
                                                    unsigned long long *gkey = nullptr) {
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, nw = blockDim.x >> 5;
  warp_argmin(ck, idx);
  if (lane == 0) {
    s_ck[warp] = ck;
    s_idx[warp] = idx;
  }
  __syncthreads();
  __shared__ bool s_last;
  if (warp == 0) {
    ck = lane < nw ? s_ck[lane] : ~0ull;
    idx = lane < nw ? s_idx[lane] : INT64_MAX;
    warp_argmin(ck, idx);
    if (lane == 0) {
      uint64_t *part = reinterpret_cast<uint64_t *>(sel + kSelPartialOff) + 2 * blockIdx.x;
      part[0] = ck;
      part[1] = (uint64_t)idx;
      __threadfence();
      unsigned int *cnt = reinterpret_cast<unsigned int *>(sel + kSelCounterOff);
      unsigned int t = atomicAdd(cnt, 1u);
      s_last = (t == gridDim.x - 1);
    }
  }
  __syncthreads();
  if (!s_last) return;
  __threadfence();
  // last CTA: reduce all partials
  const volatile uint64_t *parts = reinterpret_cast<const volatile uint64_t *>(sel + kSelPartialOff);
  ck = ~0ull;
  idx = INT64_MAX;
  for (unsigned int b = threadIdx.x; b < gridDim.x; b += blockDim.x) {
    uint64_t c2 = parts[2 * b];
    int64_t i2 = (int64_t)parts[2 * b + 1];
    if (key_less(c2, i2, ck, idx)) {
      ck = c2;
      idx = i2;
    }
  }
  warp_argmin(ck, idx);
  if (lane == 0) {
    s_ck[warp] = ck;
    s_idx[warp] = idx;
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    for (int w = 1; w < nw; ++w)
      if (key_less(s_ck[w], s_idx[w], s_ck[0], s_idx[0])) {
        s_ck[0] = s_ck[w];
        s_idx[0] = s_idx[w];
      }
    ck = s_ck[0];
    idx = s_idx[0];
    aceso_select_result *res = reinterpret_cast<aceso_select_result *>(sel);
    if (ck == ~0ull) {
      res->key = INT64_MAX;
      res->cls_cost = ~0ull;
      res->index = -1;
    } else {
      uint64_t cls = ck >> 62, cost = ck & ((1ull << 62) - 1);
      uint64_t cmax = (1ull << (62 - ib)) - 1;
      uint64_t c = cost < cmax ? cost : cmax;
      res->key = (int64_t)((cls << 62) | (c << ib) | (uint64_t)idx);
      res->cls_cost = ck;
      res->index = idx;
    }
    res->reserved = 0;
    *reinterpret_cast<unsigned int *>(sel + kSelCounterOff) = 0;  // reusable
    // global selection fused into the launch (aceso_eval_global): the packed key joins the
    // job's key by a system-scope atomic MIN on a local or NVLink peer-mapped address (the
    // key's top bit is 0, so unsigned order = signed order; "nothing valid" = INT64_MAX)
    if (gkey) atomicMin_system(gkey, (unsigned long long)res->key);
  }
}

// Argmin with grid-level completion: every warp leaves its partial in shared memory, one
// CTA barrier, warp 0 reduces the CTA's partials and publishes the CTA partial; the last
// CTA to publish (global counter) reduces all CTA partials and writes the final result.
// Called by all 32 lanes of every warp of the grid.
__device__ __forceinline__ void warp_select_finish(uint64_t ck, int64_t idx, unsigned char *sel,
                                                   int64_t n_total, uint32_t ib, uint64_t *s_ck,
                                                   int64_t *s_idx, unsigned long long *gkey = nullptr) {
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const uint32_t wpb = blockDim.x >> 5;
  warp_argmin(ck, idx);
  if (lane == 0) {
    s_ck[warp] = ck;
    s_idx[warp] = idx;
  }
  __syncthreads();
  if (warp != 0) return;
  ck = lane < (int)wpb ? s_ck[lane] : ~0ull;
  idx = lane < (int)wpb ? s_idx[lane] : INT64_MAX;
  warp_argmin(ck, idx);
  uint32_t last = 0;
  if (lane == 0) {
    uint64_t *part = reinterpret_cast<uint64_t *>(sel + kSelPartialOff) + 2 * blockIdx.x;
    part[0] = ck;
    part[1] = (uint64_t)idx;
    __threadfence();
    unsigned int *cnt = reinterpret_cast<unsigned int *>(sel + kSelCounterOff);
    last = atomicAdd(cnt, 1u) == gridDim.x - 1 ? 1u : 0u;
  }
  if (!__shfl_sync(0xffffffffu, last, 0)) return;
  __threadfence();
  const uint64_t *parts = reinterpret_cast<const uint64_t *>(sel + kSelPartialOff);
  ck = ~0ull;
  idx = INT64_MAX;
  for (uint32_t b0 = 0; b0 < gridDim.x; b0 += 32 * 8) {
    uint64_t c2[8];
    int64_t i2[8];
#pragma unroll
    for (int k = 0; k < 8; ++k) {  // 8 independent loads in flight per lane
      const uint32_t b = b0 + k * 32 + lane;
      c2[k] = b < gridDim.x ? __ldcg(parts + 2 * b) : ~0ull;
      i2[k] = b < gridDim.x ? (int64_t)__ldcg(parts + 2 * b + 1) : INT64_MAX;
    }
#pragma unroll
    for (int k = 0; k < 8; ++k)
      if (key_less(c2[k], i2[k], ck, idx)) {
        ck = c2[k];
        idx = i2[k];
      }
  }
  warp_argmin(ck, idx);
  if (lane == 0) {
    aceso_select_result *res = reinterpret_cast<aceso_select_result *>(sel);
    if (ck == ~0ull) {
      res->key = INT64_MAX;
      res->cls_cost = ~0ull;
      res->index = -1;
    } else {
      const uint64_t cls = ck >> 62, cost = ck & ((1ull << 62) - 1);
      const uint64_t cmax = (1ull << (62 - ib)) - 1;
      const uint64_t c = cost < cmax ? cost : cmax;
      res->key = (int64_t)((cls << 62) | (c << ib) | (uint64_t)idx);
      res->cls_cost = ck;
      res->index = idx;
    }
    res->reserved = 0;
    *reinterpret_cast<unsigned int *>(sel + kSelCounterOff) = 0;  // reusable
    // global selection fused into the launch (aceso_eval_global): the packed key joins the
    // job's key by a system-scope atomic MIN on a local or NVLink peer-mapped address (the
    // key's top bit is 0, so unsigned order = signed order; "nothing valid" = INT64_MAX)
    if (gkey) atomicMin_system(gkey, (unsigned long long)res->key);
  }
}

}  // namespace aceso
