// eval_kernel.cuh — batched evaluation of Aceso's performance/memory model (sm_100a).
//
// One thread per candidate configuration; a warp owns a tile of 32 candidates
// (tiled layout of include/aceso.h) and streams its 16-op chunks from HBM into a
// per-warp shared-memory ring with cp.async.bulk (TMA bulk copies, mbarrier
// completion). The packed profile tables are staged into shared memory once per
// CTA, also with cp.async.bulk. Per op the thread gathers its 16-byte record and
// the DP record from shared memory and accumulates the stage sums; stage heads and
// in-stage tp/dp changes ("events") are detected per chunk with SWAR byte tricks
// so that event-free chunks run a branch-free path. Stage close applies Eq. 1/2,
// OOM flag and Heuristic-1; the candidate epilogue writes the SoA summary and
// folds the candidate into the fused argmin (K2, common.cuh).
//
// Paper: configuration (§3.1), Heuristic-1, memory Eq. 1
// (P:L225-234), time Eq. 2; readings R1-R13 in DESIGN.md §3.
#pragma once
#include "common.cuh"

namespace aceso {

enum : uint32_t { kSummary = ACESO_OUT_SUMMARY, kFull = ACESO_OUT_FULL, kSelect = ACESO_FUSED_SELECT };

constexpr int kRingSlots = 4;    // per-warp ring depth
constexpr int kSlotChunks = 2;   // 16-op chunks per ring slot (1 KB)
constexpr int kSlotBytes = kSlotChunks * 512;
constexpr int kRingBytesPerCta = kWarps * kRingSlots * kSlotBytes;

// ---------------------------------------------------------------------------
// PTX helpers: mbarrier + cp.async.bulk (TMA bulk copy)
// ---------------------------------------------------------------------------
__device__ __forceinline__ uint32_t smem_addr(const void *p) {
  return (uint32_t)__cvta_generic_to_shared(p);
}
__device__ __forceinline__ void mbar_init(uint32_t bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(bar), "r"(count) : "memory");
}
__device__ __forceinline__ void fence_barrier_init() {
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void fence_proxy_async() {
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint32_t bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(bytes)
               : "memory");
}
__device__ __forceinline__ void bulk_g2s(uint32_t dst, const void *src, uint32_t bytes,
                                         uint32_t bar) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
          dst),
      "l"(src), "r"(bytes), "r"(bar)
      : "memory");
}
__device__ __forceinline__ void mbar_wait(uint32_t bar, uint32_t parity) {
  asm volatile(
      "{\n"
      ".reg .pred P1;\n"
      "WAIT_%=:\n"
      "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n"
      "@!P1 bra WAIT_%=;\n"
      "}\n" ::"r"(bar),
      "r"(parity)
      : "memory");
}

// shared-memory loads by absolute shared address (no generic-pointer arithmetic)
__device__ __forceinline__ uint4 lds128(const unsigned char *, uint32_t a) {
  uint4 v;
  asm volatile("ld.shared.v4.u32 {%0, %1, %2, %3}, [%4];"
               : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w)
               : "r"(a));
  return v;
}
__device__ __forceinline__ uint32_t lds32(const unsigned char *, uint32_t a) {
  uint32_t v;
  asm volatile("ld.shared.u32 %0, [%1];" : "=r"(v) : "r"(a));
  return v;
}

// ---------------------------------------------------------------------------
// per-candidate state (registers)
// ---------------------------------------------------------------------------
struct Cand {
  // current stage (per-microbatch sums, R5/R13 terms included in S)
  uint64_t S, A, W, D, comp;
  uint32_t E;
  // current run (ops with equal (tp, dp) inside one stage): absolute shared addresses,
  // kbase: offset of the run in the global cold table (16 B per type)
  uint32_t rbase, dbase, kbase, fbase, gst;
  // candidate-level
  uint64_t sumS, bestT, bestM;
  uint32_t bt, bm, oom, i, gsum, reasons, head0;
  uint32_t mbs, p;
  uint64_t N;
};

// absolute shared addresses of the staged tables
struct Smem {
  uint32_t R, D, F, T;
  const unsigned char *K;  // global cold table
};

__device__ __forceinline__ uint32_t ldk(const Smem &sm, uint32_t off) {
  return __ldg(reinterpret_cast<const uint32_t *>(sm.K + off));
}

template <uint32_t MODE>
__device__ __forceinline__ void close_stage(Cand &s, const Smem &sm, const EvalParams &P,
                                            uint32_t toff_last, int64_t c, bool active) {
  // R5: a non-last stage pays the forward send of its last op
  if (s.i + 1 < s.p) s.S += ldk(sm, s.kbase + (toff_last >> 1) + 4);
  s.sumS += s.S;
  const uint64_t tk = (s.N - 1) * s.S + s.D;  // T_i - sum_k S_k   (Eq. 2, R1, R6)
  if (s.i == 0 || tk > s.bestT) { s.bestT = tk; s.bt = s.i; }
  const uint64_t infl = s.p > s.i ? min((uint64_t)(s.p - s.i), s.N) : 0ull;  // R2
  const uint64_t M = (s.W + infl * s.A + s.E) << P.mem_shift;                 // Eq. 1
  if (s.i == 0 || M > s.bestM) { s.bestM = M; s.bm = s.i; }
  s.oom |= (M > P.C) ? 1u : 0u;  // R10
  if (MODE & kFull) {
    if (active && s.i < (uint32_t)P.p_max) {
      const int64_t o = (int64_t)s.i * P.n + c;
      P.stage_T[o] = tk;  // + sum_k S_k in the epilogue
      P.stage_mem[o] = M;
      P.stage_comp[o] = s.N * s.comp;
      P.stage_comm[o] = s.N * (s.S - s.comp) + s.D;
    }
  }
  s.i += 1;
  s.S = s.A = s.W = s.D = s.comp = 0;
  s.E = 0;
}

// Event at op j: stage head and/or change of (tp, dp). Opens the new run.
template <uint32_t MODE>
__device__ __forceinline__ void on_event(Cand &s, const Smem &sm, const EvalParams &P, uint32_t j,
                                      uint32_t c, uint32_t toff, uint32_t toff_prev, int64_t cand,
                                      bool active) {
  const uint32_t head = c & 1u;
  if (head && j > 0) close_stage<MODE>(s, sm, P, toff_prev, cand, active);
  const uint32_t tpl = (c >> 1) & 7u, dpl = c >> 5;
  if (dpl > s.mbs) s.reasons |= ACESO_R_DPMBS;
  if (tpl >= (uint32_t)P.n_tp || dpl >= (uint32_t)P.n_dp) s.reasons |= ACESO_R_TABLE;
  else if (dpl <= s.mbs && s.mbs - dpl >= (uint32_t)P.n_b) s.reasons |= ACESO_R_TABLE;
  // clamped indices keep every gather inside the tables for invalid encodings
  uint32_t b = dpl <= s.mbs ? s.mbs - dpl : 0u;
  b = min(b, (uint32_t)P.n_b - 1);
  const uint32_t tplc = min(tpl, (uint32_t)P.n_tp - 1);
  const uint32_t run = (b * (uint32_t)P.n_tp + tplc) * (uint32_t)P.T;
  s.rbase = sm.R + run * kTypeStride;
  s.kbase = run * 16u;
  if (MODE & kFull) s.fbase = sm.F + run * 8u;
  s.dbase = sm.D + tplc * (uint32_t)P.T * kTypeStride + dpl * 4u;
  const uint32_t g = tpl + dpl;
  if (head || j == 0) {
    s.gst = g;
    s.gsum += 1u << g;  // R9: sum_i tp_i * dp_i
    if (s.i > 0) s.S += ldk(sm, s.kbase + (toff >> 1) + 8);  // R5: backward send of the first op
  } else {
    if (g != s.gst) s.reasons |= ACESO_R_GSTAGE;  // P:L151 in-stage symmetry
    s.S += ldk(sm, s.kbase + (toff >> 1));       // R13: reshard into this op
  }
}

template <uint32_t MODE>
__device__ __forceinline__ void accumulate(Cand &s, const Smem &sm, uint32_t rcoff, uint32_t toff) {
  const uint32_t ra = s.rbase + toff + rcoff;
  const uint4 r = lds128(nullptr, ra);
  const uint32_t d = lds32(nullptr, s.dbase + toff);
  s.S += r.x;
  s.A += r.y;
  s.E = max(s.E, r.z);
  s.W += r.w;
  s.D += d;
  if (MODE & kFull) s.comp += lds32(nullptr, s.fbase + (toff >> 2) + (rcoff >> 2));
}

template <uint32_t MODE>
__device__ __forceinline__ void init_cand(Cand &s, const Smem &sm, const EvalParams &P, uint64_t h) {
  s.mbs = (uint32_t)(h & 0xff);
  s.p = (uint32_t)((h >> 8) & 0xff);
  s.reasons = (h >> 16) ? ACESO_R_HDR : 0u;
  s.N = 0;
  if (s.mbs >= 62 || (1ull << s.mbs) > P.Bg || (P.Bg & ((1ull << s.mbs) - 1)) != 0)
    s.reasons |= ACESO_R_MBS;
  else
    s.N = P.Bg >> s.mbs;
  if (s.p == 0 || s.p > (uint32_t)P.G) s.reasons |= ACESO_R_PRANGE;
  s.S = s.A = s.W = s.D = s.comp = 0;
  s.E = 0;
  s.sumS = s.bestT = s.bestM = 0;
  s.bt = s.bm = s.oom = s.i = s.gsum = 0;
  s.head0 = 0;
  s.rbase = sm.R;
  s.dbase = sm.D;
  s.kbase = 0;
  s.fbase = sm.F;
  s.gst = 0;
}

// Process one 16-op chunk of the lane's candidate. v = the lane's 16 code bytes.
template <uint32_t MODE>
__device__ __forceinline__ void process_chunk(Cand &s, const Smem &sm, const EvalParams &P, uint4 v,
                                              uint32_t ch, uint32_t &prevw, int64_t cand,
                                              bool active) {
  const uint32_t w[4] = {v.x, v.y, v.z, v.w};
  uint32_t x[4];
  uint32_t pw = prevw;
#pragma unroll
  for (int q = 0; q < 4; ++q) {
    // previous op's byte under each byte: funnel shift of (previous word, word)
    const uint32_t sh = __funnelshift_l(pw, w[q], 8);
    x[q] = ((w[q] ^ sh) & 0xEEEEEEEEu) | (w[q] & 0x01010101u);  // tp/dp change | head
    pw = w[q];
  }
  prevw = pw;
  const uint32_t j0 = ch * 16u;
  if (ch == 0) {
    x[0] |= 0xffu;  // op 0 always opens the first run
    s.head0 = w[0] & 1u;
  }
  const bool last = (j0 + 16u >= (uint32_t)P.L);
  const uint32_t ev = x[0] | x[1] | x[2] | x[3];
  const uint32_t ta = sm.T + j0 * 4u;  // this chunk's 16 type offsets (broadcast loads)
  if (!last && !__any_sync(0xffffffffu, ev != 0)) {
    // fast path: no head, no tp/dp change in any lane of the warp
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      const uint4 t4 = lds128(nullptr, ta + 16u * q);
      const uint32_t t[4] = {t4.x, t4.y, t4.z, t4.w};
      const uint32_t rcw = w[q] & 0x10101010u;  // rc * 16 per byte
#pragma unroll
      for (int k = 0; k < 4; ++k) accumulate<MODE>(s, sm, __byte_perm(rcw, 0, 0x4440 + k), t[k]);
    }
    return;
  }
  // general path: per-op event test
  const uint32_t kmax = last ? (uint32_t)P.L - j0 : 16u;
#pragma unroll
  for (int q = 0; q < 4; ++q) {
    uint32_t ww = w[q], xx = x[q];
#pragma unroll 1
    for (int k = 0; k < 4; ++k) {
      const uint32_t kk = 4 * q + k;
      if (kk >= kmax) break;
      const uint32_t j = j0 + kk;
      const uint32_t toff = lds32(nullptr, ta + 4u * kk);
      const uint32_t c = ww & 0xffu;
      if (xx & 0xffu) {
        const uint32_t toff_prev = j > 0 ? lds32(nullptr, ta + 4u * kk - 4u) : 0u;
        on_event<MODE>(s, sm, P, j, c, toff, toff_prev, cand, active);
      }
      accumulate<MODE>(s, sm, c & 0x10u, toff);
      ww >>= 8;
      xx >>= 8;
    }
  }
}

template <uint32_t MODE>
__device__ __forceinline__ void finish_cand(Cand &s, const Smem &sm, const EvalParams &P, int64_t c,
                                            bool active, uint64_t &best_ck, int64_t &best_idx) {
  close_stage<MODE>(s, sm, P, lds32(nullptr, sm.T + 4u * (uint32_t)(P.L - 1)), c, active);
  const uint32_t nheads = s.i - 1 + s.head0;
  if (!s.head0) s.reasons |= ACESO_R_HEAD0;
  if (nheads != s.p) s.reasons |= ACESO_R_NSTAGE;
  if (s.gsum != (uint32_t)P.G) s.reasons |= ACESO_R_GSUM;
  const bool invalid = s.reasons != 0;
  const uint64_t iter = invalid ? 0ull : s.sumS + s.bestT;  // max_i T_i (Eq. 2)
  const uint64_t mem = invalid ? 0ull : s.bestM;
  uint32_t info = (s.p << 8);
  if (invalid) info |= ACESO_INFO_INVALID | (s.reasons << 18);
  else info |= (s.oom ? (s.bm | ACESO_INFO_OOM) : s.bt);  // Heuristic-1
  if (active) {
    if (MODE & kSummary) {
      P.iter_ns[c] = iter;
      P.max_mem[c] = mem;
      P.info[c] = info;
    }
    if ((MODE & kFull) && !invalid) {
      const uint32_t ns = min(s.i, (uint32_t)P.p_max);
      for (uint32_t k = 0; k < ns; ++k) P.stage_T[(int64_t)k * P.n + c] += s.sumS;
    }
    if ((MODE & kSelect) && !invalid) {
      // class 0 feasible (cost = iteration time), class 1 OOM (cost = max memory), R12
      const uint64_t ck = s.oom ? ((1ull << 62) | mem) : iter;
      const int64_t g = P.gofs + c;
      if (key_less(ck, g, best_ck, best_idx)) {
        best_ck = ck;
        best_idx = g;
      }
    }
  }
}

template <uint32_t MODE>
__global__ void __launch_bounds__(kThreads) eval_kernel(const __grid_constant__ EvalParams P) {
  extern __shared__ __align__(128) unsigned char sm_raw[];
  __shared__ __align__(8) uint64_t s_tbar;
  __shared__ __align__(8) uint64_t s_ring_bar[kWarps][kRingSlots];
  __shared__ uint64_t s_ck[kWarps];
  __shared__ int64_t s_idx[kWarps];

  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const uint32_t tab_bytes = (MODE & kFull) ? P.tab.bytes_full : P.tab.bytes;
  const uint32_t sb = smem_addr(sm_raw);
  Smem sm;
  sm.R = sb + P.tab.offR;
  sm.D = sb + P.tab.offD;
  sm.T = sb + P.tab.offT;
  sm.F = sb + P.tab.offF;
  sm.K = reinterpret_cast<const unsigned char *>(P.blob) + P.tab.offK;
  const uint32_t ring = sb + tab_bytes + (uint32_t)warp * kRingSlots * kSlotBytes;

  // ---- stage the packed tables (one bulk copy, TMA) ----
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
    mbar_expect_tx(bar, tab_bytes);
    bulk_g2s(sb, P.blob, tab_bytes, bar);
  }

  // ---- this warp's stream of units (tile, group of kSlotChunks chunks) ----
  const int64_t first_tile = (int64_t)blockIdx.x * kWarps + warp;
  const int64_t tile_stride = (int64_t)gridDim.x * kWarps;
  const int64_t my_tiles =
      first_tile < P.n_tiles ? (P.n_tiles - first_tile + tile_stride - 1) / tile_stride : 0;
  const uint32_t ngroups = ((uint32_t)P.nch + kSlotChunks - 1) / kSlotChunks;
  const int64_t units = my_tiles * ngroups;

  auto issue = [&](int64_t u) {
    const int64_t t = first_tile + (u / ngroups) * tile_stride;
    const uint32_t g = (uint32_t)(u % ngroups);
    const uint32_t c0 = g * kSlotChunks;
    const uint32_t nc = min((uint32_t)kSlotChunks, (uint32_t)P.nch - c0);
    const int slot = (int)(u % kRingSlots);
    const uint32_t bar = smem_addr(&s_ring_bar[warp][slot]);
    const unsigned char *src =
        reinterpret_cast<const unsigned char *>(P.codes) + ((size_t)t * P.nch + c0) * 512;
    mbar_expect_tx(bar, nc * 512u);
    bulk_g2s(ring + slot * kSlotBytes, src, nc * 512u, bar);
  };
  if (lane == 0) {
    for (int64_t u = 0; u < units && u < kRingSlots; ++u) issue(u);
  }
  __syncwarp();

  mbar_wait(smem_addr(&s_tbar), 0);  // tables resident

  uint64_t best_ck = ~0ull;
  int64_t best_idx = INT64_MAX;
  Cand s;
  uint32_t prevw = 0;
  int64_t cand = 0;
  bool active = false;
  for (int64_t u = 0; u < units; ++u) {
    const int64_t t = first_tile + (u / ngroups) * tile_stride;
    const uint32_t g = (uint32_t)(u % ngroups);
    const int slot = (int)(u % kRingSlots);
    if (g == 0) {
      cand = t * 32 + lane;
      active = cand < P.n;
      init_cand<MODE>(s, sm, P, active ? __ldg(P.hdr + cand) : 0ull);
      prevw = 0;
    }
    mbar_wait(smem_addr(&s_ring_bar[warp][slot]), (uint32_t)((u / kRingSlots) & 1));
    const uint32_t c0 = g * kSlotChunks;
    const uint32_t nc = min((uint32_t)kSlotChunks, (uint32_t)P.nch - c0);
    const uint32_t slot_a = ring + slot * kSlotBytes + lane * 16;
    for (uint32_t k = 0; k < nc; ++k) {
      const uint4 v = lds128(nullptr, slot_a + k * 512);
      process_chunk<MODE>(s, sm, P, v, c0 + k, prevw, cand, active);
    }
    __syncwarp();
    if (lane == 0 && u + kRingSlots < units) {
      fence_proxy_async();
      issue(u + kRingSlots);
    }
    if (g == ngroups - 1) finish_cand<MODE>(s, sm, P, cand, active, best_ck, best_idx);
  }

  if (MODE & kSelect)
    block_select_finish(best_ck, best_idx, P.sel, P.n_total, P.ib, s_ck, s_idx);
}

}  // namespace aceso
