// dense_kernel.cuh — per-op evaluation for candidates whose tp/dp changes at most ops
// (ACESO_HINT_DENSE; e.g. uniformly random encodings), sm_100a.
//
// Same contract, records and outputs as eval_kernel.cuh (thread = candidate, warp = tile of
// 32 candidates streamed through a per-warp cp.async.bulk ring, profile tables staged in
// shared memory, here TYPE-major: the 32 lanes evaluate the same op, so they read one type's
// records of different runs — neighbouring 32-byte records instead of one bank every
// T x 32 bytes), but no event handler: every op is accumulated by the same branch-free
// sequence under its OWN (b, tp) record — so an in-stage tp/dp change costs one predicated
// reshard lookup instead of a run switch, and lanes stay converged except at stage heads
// (at most p per candidate).
//
// Per op j with code c (head, log2 tp, recompute, log2 dp):
//   head at j > 0 : the open stage takes p2p_fwd of op j-1 (R5) and closes (Eq. 1/2, OOM,
//                   Heuristic-1: stage_commit); the new stage takes p2p_bwd of op j (R5)
//   otherwise     : reshard of op j if its (tp, dp) differs from op j-1's (R13);
//                   tp*dp must equal the stage's (R9)
//   every op      : S += fwd+bwd (+fwd if rc, R7), A += act or keep (R3),
//                   E = max(E, peak (+act-keep if rc)) (R4), W += param+opt, D += DP sync (R6)
// Readings R1-R13, R18-R20 in DESIGN.md §3.
//
// Tensor-parallel partition dimension (§4.2): with DIMS the candidates carry a
// dimension bit per op (aceso_eval_dims); an op on its alternative dimension reads the records
// of type + T (the tables then hold 2T types: the alternative dimension's records, same
// parameter and DP-sync entries). GT: the tables stay in global memory (L2) when they do not
// fit shared memory (e.g. Wide-ResNet with alternative records).
#pragma once
#include <type_traits>

#include "eval_kernel.cuh"

namespace aceso {

// table accessors: shared memory (staged once per CTA) or global memory (L2-resident)
struct DTabS {
  uint32_t b;
  __device__ __forceinline__ uint32_t u32(uint32_t o) const { return lds32(b + o); }
  __device__ __forceinline__ uint2 u64(uint32_t o) const { return lds64(b + o); }
  __device__ __forceinline__ uint4 u128(uint32_t o) const { return lds128(b + o); }
};
struct DTabG {
  const unsigned char *b;
  __device__ __forceinline__ uint32_t u32(uint32_t o) const { return __ldg(reinterpret_cast<const uint32_t *>(b + o)); }
  __device__ __forceinline__ uint2 u64(uint32_t o) const { return __ldg(reinterpret_cast<const uint2 *>(b + o)); }
  __device__ __forceinline__ uint4 u128(uint32_t o) const { return __ldg(reinterpret_cast<const uint4 *>(b + o)); }
};

template <uint32_t MODE, int MINB, bool DIMS = false, bool GT = false>
__global__ void __launch_bounds__(kThreads, MINB) dense_kernel(const __grid_constant__ EvalParams P) {
  extern __shared__ __align__(128) unsigned char sm_raw[];
  __shared__ __align__(8) uint64_t s_tbar;
  __shared__ __align__(8) uint64_t s_ring_bar[kWarps][kRingSlots];
  __shared__ uint64_t s_ck[kWarps];
  __shared__ int64_t s_idx[kWarps];

  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const uint32_t stage_bytes = GT ? 0u : (MODE & kFull) ? P.tab.dbytes_full : P.tab.dbytes;
  const uint32_t sb = smem_addr(sm_raw);
  typename std::conditional<GT, DTabG, DTabS>::type tb;
  if constexpr (GT) tb.b = reinterpret_cast<const unsigned char *>(P.blob) + P.tab.dOff;
  else tb.b = sb;
  const uint32_t DR = P.tab.dR, DD = P.tab.dD, DK = P.tab.dK, DT = P.tab.dT, DF = P.tab.dF;
  const uint32_t T = (uint32_t)P.T;  // alternative-dimension records: type + T
  const uint32_t runs = (uint32_t)(P.n_b * P.n_tp);
  const uint32_t ring = sb + stage_bytes + (uint32_t)warp * kRingSlots * kSlotBytes;
  Smem sm;  // init_cand's table bases (unused here)
  sm.R = sm.D = sm.F = sm.QT = sm.QD = sm.QF = sb;

  if (threadIdx.x == 0) {
    mbar_init(smem_addr(&s_tbar), 1);
    fence_barrier_init();
  }
  if (lane == 0) {
    for (int k = 0; k < kRingSlots; ++k) mbar_init(smem_addr(&s_ring_bar[warp][k]), 1);
    fence_barrier_init();
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    const uint32_t bar = smem_addr(&s_tbar);
    if (GT) {
      asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(bar) : "memory");
    } else {
      mbar_expect_tx(bar, stage_bytes);
      bulk_g2s(sb, reinterpret_cast<const unsigned char *>(P.blob) + P.tab.dOff, stage_bytes, bar);
    }
  }

  const uint32_t nch = (uint32_t)P.nch;
  const uint32_t L = (uint32_t)P.L;
  const uint32_t ngroups = (nch + kSlotChunks - 1) / kSlotChunks;
  const int64_t first_tile = (int64_t)blockIdx.x * kWarps + warp;
  const int64_t tile_stride = (int64_t)gridDim.x * kWarps;
  const int64_t my_tiles = first_tile < P.n_tiles ? (P.n_tiles - first_tile + tile_stride - 1) / tile_stride : 0;
  const int64_t units = my_tiles * ngroups;
  const unsigned char *codes = reinterpret_cast<const unsigned char *>(P.codes);

  int64_t it_tile = first_tile;
  uint32_t it_g = 0;
  auto issue_next = [&](int slot) {
    const uint32_t a = kSlotChunks * it_g, b = min(a + kSlotChunks, nch);
    const uint32_t bar = smem_addr(&s_ring_bar[warp][slot]);
    mbar_expect_tx(bar, (b - a) * 512u);
    bulk_g2s(ring + slot * kSlotBytes, codes + ((size_t)it_tile * nch + a) * 512, (b - a) * 512u, bar);
    if (++it_g == ngroups) {
      it_g = 0;
      it_tile += tile_stride;
    }
  };
  if (lane == 0) {
    for (int64_t u = 0; u < units && u < kRingSlots; ++u) issue_next((int)u);
  }
  __syncwarp();
  mbar_wait(smem_addr(&s_tbar), 0);  // tables resident

  const uint32_t n_tp = (uint32_t)P.n_tp, n_dp = (uint32_t)P.n_dp, n_b = (uint32_t)P.n_b;
  uint64_t best_ck = ~0ull;
  int64_t best_idx = INT64_MAX;
  Cand s = Cand();
  uint32_t prev = 0;   // code of op j-1
  uint32_t pk = 0;     // shared address of op j-1's DK record (its run and type)
  int64_t tile = first_tile;
  uint32_t g = 0;
  int slot = 0;
  uint32_t phase = 0;
  int64_t cand = 0;
  bool active = false;
  // table-range validity (R18 DPMBS / TABLE) depends only on the extremes of tp and dp over
  // the candidate's ops: tracked per op, decided once per candidate
  uint32_t max_tpl = 0, max_dpl = 0, min_dpl = 7;
  // one op (j, code c, type ty): the accumulation described at the top of the file
  auto op = [&](uint32_t j, uint32_t c, uint32_t ty) {
    const uint32_t tpl = (c >> 1) & 7u, dpl = c >> 5, rc = (c >> 4) & 1u;
    const uint32_t gg = tpl + dpl;
    max_tpl = max(max_tpl, tpl);
    max_dpl = max(max_dpl, dpl);
    min_dpl = min(min_dpl, dpl);
    // clamped indices keep every gather inside the tables for invalid encodings
    const uint32_t bb = min(dpl <= s.mbs ? s.mbs - dpl : 0u, n_b - 1u);
    const uint32_t tplc = min(tpl, n_tp - 1u);
    const uint32_t tr = ty * runs + bb * n_tp + tplc;  // (type, run) record index
    const uint32_t kofs = DK + tr * 16u;
    if ((c & 1u) || j == 0) {
      if ((c & 1u) && j > 0) {
        s.S += tb.u32(pk + 4u);  // R5: p2p_fwd of the stage's last op (j-1)
        stage_commit<MODE>(s, P, cand, active);
        s.i += 1;
        s.S += tb.u32(kofs + 8u);  // R5: p2p_bwd of the stage's first op
      }
      s.gst = gg;
      s.gsum += 1u << gg;  // R9
      s.nheads += c & 1u;
    } else {
      if (gg != s.gst) s.reasons |= ACESO_R_GSTAGE;  // P:L151 in-stage symmetry
      if ((c ^ prev) & 0xeeu) s.S += tb.u32(kofs);     // R13: reshard into op j
    }
    const uint4 r = tb.u128(DR + tr * 32u + rc * 16u);
    s.S += r.x;
    s.A += r.y;
    s.E = max(s.E, r.z);
    s.W += r.w;
    s.D += tb.u32(DD + (ty * n_tp + tplc) * 32u + dpl * 4u);
    if (MODE & kFull) s.comp += tb.u32(DF + tr * 8u + rc * 4u);
    prev = c;
    pk = kofs;
  };
  for (int64_t u = 0; u < units; ++u) {
    if (g == 0) {
      cand = tile * 32 + lane;
      active = cand < P.n;
      init_cand(s, sm, P, active ? __ldg(P.hdr + cand) : 0ull);
      max_tpl = max_dpl = 0;
      min_dpl = 7;
    }
    mbar_wait(smem_addr(&s_ring_bar[warp][slot]), phase);
    const uint32_t a = kSlotChunks * g, b = min(a + kSlotChunks, nch);
    const uint32_t slot_a = ring + slot * kSlotBytes + lane * 16;
    if (g == 0) s.head0 = lds32(slot_a) & 1u;
#pragma unroll 1
    for (uint32_t ch = a; ch < b; ++ch) {
      const uint4 w4 = lds128(slot_a + (ch - a) * 512u);
      // dimension bits of the chunk's 16 ops (bit k = op 16 ch + k): alternative type = type + T
      uint32_t dm = 0;
      if (DIMS)
        dm = __ldg(reinterpret_cast<const unsigned short *>(P.dims + ((size_t)tile * nch + ch) * 64u) + lane);
      const uint32_t nq = min(4u, (L - ch * 16u + 3u) >> 2);  // quads inside L
#pragma unroll 1
      for (uint32_t q = 0; q < nq; ++q) {
        const uint32_t w = q == 0 ? w4.x : q == 1 ? w4.y : q == 2 ? w4.z : w4.w;
        const uint32_t j0 = ch * 16u + q * 4u;
        const uint2 tt = tb.u64(DT + 2u * j0);  // the quad's 4 u16 types
        const uint32_t dq = DIMS ? (dm >> (4u * q)) & 0xfu : 0u;
        if (j0 + 4u <= L) {  // full quad
          op(j0, w & 0xffu, (tt.x & 0xffffu) + (dq & 1u) * T);
          op(j0 + 1u, (w >> 8) & 0xffu, (tt.x >> 16) + ((dq >> 1) & 1u) * T);
          op(j0 + 2u, (w >> 16) & 0xffu, (tt.y & 0xffffu) + ((dq >> 2) & 1u) * T);
          op(j0 + 3u, w >> 24, (tt.y >> 16) + (dq >> 3) * T);
        } else {
#pragma unroll 1
          for (uint32_t k = 0; j0 + k < L; ++k)
            op(j0 + k, (w >> (8u * k)) & 0xffu,
               ((k < 2 ? tt.x >> (16u * k) : tt.y >> (16u * (k - 2))) & 0xffffu) + ((dq >> k) & 1u) * T);
        }
      }
    }
    __syncwarp();
    if (lane == 0 && u + kRingSlots < units) {
      fence_proxy_async();
      issue_next(slot);
    }
    slot = (slot + 1) % kRingSlots;
    if (slot == 0) phase ^= 1u;
    if (++g == ngroups) {
      if (max_dpl > s.mbs) s.reasons |= ACESO_R_DPMBS;
      if (max_tpl >= n_tp || max_dpl >= n_dp || (min_dpl <= s.mbs && s.mbs - min_dpl >= n_b))
        s.reasons |= ACESO_R_TABLE;
      stage_commit<MODE>(s, P, cand, active);  // last stage: no p2p_fwd
      finish_cand<MODE>(s, P, cand, active, best_ck, best_idx);
      g = 0;
      tile += tile_stride;
    }
  }

  if (MODE & kSelect) block_select_finish(best_ck, best_idx, P.sel, P.n_total, P.ib, s_ck, s_idx, P.gkey);
}

}  // namespace aceso
