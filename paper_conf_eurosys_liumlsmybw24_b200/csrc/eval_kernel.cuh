// eval_kernel.cuh — batched evaluation of Aceso's performance/memory model (sm_100a).
//
// Work decomposition. A tile holds 32 candidates (tiled layout of include/aceso.h);
// thread = candidate, one warp walks a tile's ops forward. (Round 1 also built a warp-pair
// variant, one warp walking the second half of the ops backward; measured slower and
// removed in round 2.)
//
// Data movement. The packed profile tables are staged into shared memory once per
// CTA with one cp.async.bulk (TMA bulk copy, mbarrier completion); each warp streams
// its chunks (512 B = 32 candidates x 16 ops) from HBM into a private 4-slot ring
// with cp.async.bulk, so loads run several chunks ahead of the math.
//
// Per op. A 16-byte record {S', A, e, W} is gathered from shared memory at
// run_base + type_offset + rc*16 plus the DP record; the sums are u64. Stage heads
// and in-stage tp/dp changes ("events") are detected per chunk with SWAR byte
// tricks and OR-reduced across the warp; a 4-op group without events in any lane
// runs branch-free, otherwise each op tests the warp-uniform union and only lanes
// with an event run the handler (stage close: Eq. 1/2, OOM, Heuristic-1 bookkeeping;
// run open: validity, table bases, reshard / p2p terms).
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
constexpr uint32_t kNone = 0xffffffffu;


// ---------------------------------------------------------------------------
// PTX helpers: mbarrier + cp.async.bulk (TMA bulk copy), shared loads
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
__device__ __forceinline__ uint4 lds128(uint32_t a) {
  uint4 v;
  asm volatile("ld.shared.v4.u32 {%0, %1, %2, %3}, [%4];"
               : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w)
               : "r"(a));
  return v;
}
__device__ __forceinline__ uint32_t lds32(uint32_t a) {
  uint32_t v;
  asm volatile("ld.shared.u32 %0, [%1];" : "=r"(v) : "r"(a));
  return v;
}
__device__ __forceinline__ uint2 lds64(uint32_t a) {
  uint2 v;
  asm volatile("ld.shared.v2.u32 {%0, %1}, [%2];" : "=r"(v.x), "=r"(v.y) : "r"(a));
  return v;
}
__device__ __forceinline__ uint32_t lds16(uint32_t a) {
  uint16_t v;
  asm volatile("ld.shared.u16 %0, [%1];" : "=h"(v) : "r"(a));
  return v;
}
// type offset (type * 32) of op j from the u16 type table
__device__ __forceinline__ uint32_t toff_of(uint32_t T, uint32_t j) { return lds16(T + 2u * j) << 5; }

// ---------------------------------------------------------------------------
// state
// ---------------------------------------------------------------------------
struct Smem {
  uint32_t R, D, F, T, K;   // shared addresses of the staged tables (K valid if k_smem)
  uint32_t QO, QT, QD, QF;  // quad tables: per-quad offsets, sums, DP sums, comp sums
  const unsigned char *Kg;  // cold table in global memory
  uint32_t k_smem;
  uint32_t TS;              // T * 32: bytes of one (b, tpl) block of R
};

__device__ __forceinline__ uint32_t ldk(const Smem &sm, uint32_t off) {
  return sm.k_smem ? lds32(sm.K + off) : __ldg(reinterpret_cast<const uint32_t *>(sm.Kg + off));
}

struct Cand {
  // current stage: per-microbatch sums (R5/R13 terms included in S)
  uint64_t S, A, W, D, comp;
  uint32_t E;
  // current run (ops of equal (tp, dp) inside one stage): per-op and per-quad table bases
  uint32_t rbase, dbase, kbase, fbase, gst;
  uint32_t qrun, qd, qf;
  // candidate-level aggregates
  uint64_t sumS, bestT, bestM;
  uint32_t bt, bm, oom, i, gsum, reasons, nheads, head0;
  uint32_t mbs, p, N;
};

// Closes the current stage i: Eq. 2 key, Eq. 1 memory, OOM, Heuristic-1 maxima.
template <uint32_t MODE, class St>
__device__ __forceinline__ void stage_commit(St &s, const EvalParams &P, int64_t c, bool active) {
  s.sumS += s.S;
  const uint64_t tk = (uint64_t)(s.N - P.n_minus) * s.S + s.D;  // T_i - sum_k S_k (Eq. 2, R1, R6)
  const uint64_t infl = s.p > s.i ? (uint64_t)min(s.p - s.i, s.N) : 0ull;  // R2
  const uint64_t M = (s.W + infl * s.A + s.E) << P.mem_shift;              // Eq. 1 (R3, R4)
  // argmax with the lowest stage index on ties (R11): ascending indices, strict >
  if (tk > s.bestT) { s.bestT = tk; s.bt = s.i; }
  if (M > s.bestM) { s.bestM = M; s.bm = s.i; }
  s.oom |= (M > P.C) ? 1u : 0u;  // R10
  if (MODE & kFull) {
    if (active && s.i < (uint32_t)P.p_max) {
      const int64_t o = (int64_t)s.i * P.n + c;
      P.stage_T[o] = tk;  // + sum_k S_k in the epilogue
      P.stage_mem[o] = M;
      P.stage_comp[o] = (uint64_t)s.N * s.comp;
      P.stage_comm[o] = (uint64_t)s.N * (s.S - s.comp) + s.D;
    }
  }
  s.S = s.A = s.W = s.D = s.comp = 0;
  s.E = 0;
}

// Opens the run of op code c: validity checks and table bases for its (tp, dp).
template <uint32_t MODE>
__device__ __forceinline__ void open_run(Cand &s, const Smem &sm, const EvalParams &P, uint32_t c) {
  const uint32_t tpl = (c >> 1) & 7u, dpl = c >> 5;
  if (dpl > s.mbs) s.reasons |= ACESO_R_DPMBS;
  const bool tab = tpl >= (uint32_t)P.n_tp || dpl >= (uint32_t)P.n_dp ||
                   (dpl <= s.mbs && s.mbs - dpl >= (uint32_t)P.n_b);
  if (tab) s.reasons |= ACESO_R_TABLE;
  // clamped indices keep every gather inside the tables for invalid encodings
  const uint32_t b = min(dpl <= s.mbs ? s.mbs - dpl : 0u, (uint32_t)P.n_b - 1);
  const uint32_t tplc = min(tpl, (uint32_t)P.n_tp - 1);
  const uint32_t run = b * (uint32_t)P.n_tp + tplc;
  s.rbase = sm.R + run * sm.TS;
  s.kbase = run * (sm.TS >> 1);
  if (MODE & kFull) s.fbase = sm.F + run * (sm.TS >> 2);
  s.dbase = sm.D + tplc * sm.TS + dpl * 4u;
  s.qrun = sm.QT + run * 32u;
  s.qd = sm.QD + tplc * 32u + dpl * 4u;
  if (MODE & kFull) s.qf = sm.QF + run * 8u;
}

// a whole quad from the quad tables: o = {sig * quad-sum stride, sig * DP stride},
// rsel = rc * 16 (uniform rc inside the quad)
template <uint32_t MODE>
__device__ __forceinline__ void accumulate_quad(Cand &s, uint2 o, uint32_t rsel) {
  const uint4 r = lds128(s.qrun + o.x + rsel);
  const uint32_t d = lds32(s.qd + o.y);
  s.S += r.x;
  s.A += r.y;
  s.E = max(s.E, r.z);
  s.W += r.w;
  s.D += d;
  if (MODE & kFull) s.comp += lds32(s.qf + (o.x >> 2) + (rsel >> 2));
}

template <uint32_t MODE>
__device__ __forceinline__ void accumulate(Cand &s, uint32_t rcoff, uint32_t toff) {
  const uint32_t ra = s.rbase + toff + rcoff;
  const uint4 r = lds128(ra);
  const uint32_t d = lds32(s.dbase + toff);
  s.S += r.x;
  s.A += r.y;
  s.E = max(s.E, r.z);
  s.W += r.w;
  s.D += d;
  if (MODE & kFull) s.comp += lds32(s.fbase + (toff >> 2) + (rcoff >> 2));
}

// forward event at op j (before accumulating op j): stage head and/or tp/dp change
template <uint32_t MODE>
__device__ __forceinline__ void fwd_event(Cand &s, const Smem &sm, const EvalParams &P, uint32_t j,
                                          uint32_t c, uint32_t toff, uint32_t toff_prev, int64_t cand,
                                          bool active) {
  const uint32_t head = c & 1u;
  if (head && j > 0) {
    s.S += ldk(sm, s.kbase + (toff_prev >> 1) + 4);  // R5: p2p_fwd of the stage's last op
    stage_commit<MODE>(s, P, cand, active);
    s.i += 1;
  }
  const uint32_t g = ((c >> 1) & 7u) + (c >> 5);
  open_run<MODE>(s, sm, P, c);
  if (head || j == 0) {
    s.gst = g;
    s.gsum += 1u << g;  // R9
    s.nheads += head;
    if (head && j > 0) s.S += ldk(sm, s.kbase + (toff >> 1) + 8);  // R5: p2p_bwd of the first op
  } else {
    if (g != s.gst) s.reasons |= ACESO_R_GSTAGE;  // P:L151 in-stage symmetry
    s.S += ldk(sm, s.kbase + (toff >> 1));        // R13: reshard into this op
  }
}

__device__ __forceinline__ void init_cand(Cand &s, const Smem &sm, const EvalParams &P, uint64_t h) {
  s.mbs = (uint32_t)(h & 0xff);
  s.p = (uint32_t)((h >> 8) & 0xff);
  s.reasons = (h >> 16) ? ACESO_R_HDR : 0u;
  s.N = 0;
  if (s.mbs >= 62 || (1ull << s.mbs) > P.Bg || (P.Bg & ((1ull << s.mbs) - 1)) != 0)
    s.reasons |= ACESO_R_MBS;
  else
    s.N = (uint32_t)(P.Bg >> s.mbs);
  if (s.p == 0 || s.p > (uint32_t)P.G) s.reasons |= ACESO_R_PRANGE;
  s.S = s.A = s.W = s.D = s.comp = 0;
  s.E = 0;
  s.sumS = s.bestT = s.bestM = 0;
  s.bt = s.bm = 0u;
  s.oom = s.gsum = s.nheads = s.head0 = 0;
  s.i = 0u;
  s.rbase = sm.R;
  s.dbase = sm.D;
  s.kbase = 0;
  s.fbase = sm.F;
  s.qrun = sm.QT;
  s.qd = sm.QD;
  s.qf = sm.QF;
  s.gst = 0;
}

// ---------------------------------------------------------------------------
// 4-op groups ("quads"): the unit of the event test. One call site keeps the kernel
// small enough for the instruction cache.
// ---------------------------------------------------------------------------
// forward quad qg (ops 4qg..4qg+3); w = the lane's 4 code bytes; pw = previous word
template <uint32_t MODE>
__device__ __forceinline__ void quad_fwd(Cand &s, const Smem &sm, const EvalParams &P, uint32_t w,
                                         uint2 o, uint32_t &pw, uint32_t qg, int64_t cand,
                                         bool active) {
  const uint32_t sh = __funnelshift_l(pw, w, 8);  // previous op's byte under each byte
  // per byte: bit 0 = head; bits 1-7 = difference to the previous op's code. For op 0 of
  // a tile the caller seeds pw so that op 0 always shows a tp/dp difference (opens a run).
  uint32_t d;
  asm("lop3.b32 %0, %1, %2, %3, 0xB4;" : "=r"(d) : "r"(w), "r"(sh), "r"(0x01010101u));  // c ? w : w^sh
  d &= 0xffffffefu;  // an rc change at the quad's first op does not make it mixed
  pw = w;
  // clean lane (no head, no tp/dp change, uniform rc) -> one quad-table gather
  if (d == 0u && o.x != kNone) {
    accumulate_quad<MODE>(s, o, w & 0x10u);
    return;
  }
  const uint32_t x = d & 0xefefefefu;  // events: head or tp/dp change
  const uint32_t j0 = qg * 4u;
  const uint32_t nvalid = min(4u, (uint32_t)P.L - j0);
  const uint2 tt = lds64(sm.T + 2u * j0);  // the quad's 4 u16 types
  const uint32_t t4[4] = {(tt.x & 0xffffu) << 5, (tt.x >> 16) << 5, (tt.y & 0xffffu) << 5,
                          (tt.y >> 16) << 5};
  const uint32_t rc4 = w & 0x10101010u;
#pragma unroll
  for (int k = 0; k < 4; ++k) {
    if ((uint32_t)k < nvalid) {
      if ((x >> (8 * k)) & 0xffu) {
        const uint32_t tprev = k > 0 ? t4[k - 1] : (j0 > 0 ? toff_of(sm.T, j0 - 1) : 0u);
        fwd_event<MODE>(s, sm, P, j0 + k, (w >> (8 * k)) & 0xffu, t4[k], tprev, cand, active);
      }
      accumulate<MODE>(s, __byte_perm(rc4, 0, 0x4440 + k), t4[k]);
    }
  }
}

// Candidate epilogue: validity, summary outputs, fused argmin.
template <uint32_t MODE, class St>
__device__ __forceinline__ void finish_cand(St &s, const EvalParams &P, int64_t c, bool active,
                                            uint64_t &best_ck, int64_t &best_idx) {
  if (!s.head0) s.reasons |= ACESO_R_HEAD0;
  if (s.nheads != s.p) s.reasons |= ACESO_R_NSTAGE;
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
      const uint32_t ns = min(s.p, (uint32_t)P.p_max);
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

// ---------------------------------------------------------------------------
// kernel
// ---------------------------------------------------------------------------
// MINB: resident CTAs per SM the register allocation targets (2: ~96 registers, lowest
// latency per launch; 3: <= 80 registers, more warps when independent batches overlap)
template <uint32_t MODE, int MINB>
__global__ void __launch_bounds__(kThreads, MINB) eval_kernel(const __grid_constant__ EvalParams P) {
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
  sm.QO = sb + P.tab.offQO;
  sm.QT = sb + P.tab.offQT;
  sm.QD = sb + P.tab.offQD;
  sm.QF = sb + P.tab.offQF;
  sm.K = sb + tab_bytes;  // cold table staged after the other tables when k_smem
  sm.Kg = reinterpret_cast<const unsigned char *>(P.blob) + P.tab.offK;
  sm.k_smem = P.tab.k_smem;
  sm.TS = (uint32_t)P.T * kTypeStride;
  const uint32_t stage_bytes = tab_bytes + (P.tab.k_smem ? P.tab.bytesK : 0u);
  const uint32_t ring = sb + stage_bytes + (uint32_t)warp * kRingSlots * kSlotBytes;

  // ---- stage the packed tables (TMA bulk copies) ----
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
    mbar_expect_tx(bar, stage_bytes);
    bulk_g2s(sb, P.blob, tab_bytes, bar);
    if (P.tab.k_smem) bulk_g2s(sb + tab_bytes, sm.Kg, P.tab.bytesK, bar);
  }

  // ---- every tile this warp owns ----
  const uint32_t nch = (uint32_t)P.nch;
  const uint32_t ngroups = (nch + kSlotChunks - 1) / kSlotChunks;
  const int64_t first_tile = (int64_t)blockIdx.x * kWarps + warp;
  const int64_t tile_stride = (int64_t)gridDim.x * kWarps;
  const int64_t my_tiles =
      first_tile < P.n_tiles ? (P.n_tiles - first_tile + tile_stride - 1) / tile_stride : 0;
  const int64_t units = my_tiles * ngroups;
  const unsigned char *codes = reinterpret_cast<const unsigned char *>(P.codes);

  // chunk range of group g
  auto group_lo = [&](uint32_t g) { return kSlotChunks * g; };
  auto group_hi = [&](uint32_t g) { return min(kSlotChunks * (g + 1), nch); };
  // issue cursor (lane 0)
  int64_t it_tile = first_tile;
  uint32_t it_g = 0;
  auto issue_next = [&](int slot) {
    const uint32_t a = group_lo(it_g), b = group_hi(it_g);
    const uint32_t bar = smem_addr(&s_ring_bar[warp][slot]);
    mbar_expect_tx(bar, (b - a) * 512u);
    bulk_g2s(ring + slot * kSlotBytes, codes + ((size_t)it_tile * nch + a) * 512, (b - a) * 512u,
             bar);
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

  uint64_t best_ck = ~0ull;
  int64_t best_idx = INT64_MAX;
  Cand s;
  uint32_t cw = 0;  // the previous code word
  int64_t tile = first_tile;
  uint32_t g = 0;
  int slot = 0;
  uint32_t phase = 0;
  int64_t cand = 0;
  bool active = false;
  for (int64_t u = 0; u < units; ++u) {
    if (g == 0) {
      cand = tile * 32 + lane;
      active = cand < P.n;
      init_cand(s, sm, P, active ? __ldg(P.hdr + cand) : 0ull);
      cw = 0;
    }
    mbar_wait(smem_addr(&s_ring_bar[warp][slot]), phase);
    const uint32_t a = group_lo(g), b = group_hi(g);
    const uint32_t slot_a = ring + slot * kSlotBytes + lane * 16;
    if (g == 0) {
      // seed the previous word so that op 0 always opens the first run
      const uint32_t w0 = lds32(slot_a);
      cw = ((w0 & 0xffu) ^ 0x02u) << 24;
      s.head0 = w0 & 1u;
    }
#pragma unroll 1
    for (uint32_t ch = a; ch < b; ++ch) {
      const uint32_t nqc = min(4u, ((uint32_t)P.L - ch * 16u + 3u) >> 2);  // quads inside L
      uint32_t wa = slot_a + (ch - a) * 512u;
      uint32_t oa = sm.QO + 8u * (ch * 4u);
      // software pipeline: the next quad's code word and signature offsets load while
      // this quad is processed
      uint32_t wn = lds32(wa);
      uint2 on = lds64(oa);
#pragma unroll 1
      for (uint32_t q = 0; q < nqc; ++q) {
        const uint32_t w = wn;
        const uint2 o = on;
        wa += 4u;
        oa += 8u;
        if (q + 1 < nqc) {
          wn = lds32(wa);
          on = lds64(oa);
        }
        quad_fwd<MODE>(s, sm, P, w, o, cw, ch * 4u + q, cand, active);
      }
    }
    __syncwarp();
    if (lane == 0 && u + kRingSlots < units) {
      fence_proxy_async();
      issue_next(slot);
    }
    if (++slot == kRingSlots) {
      slot = 0;
      phase ^= 1u;
    }
    if (++g == ngroups) {
      // ---- tile epilogue ----
      stage_commit<MODE>(s, P, cand, active);  // last stage: no p2p_fwd
      finish_cand<MODE>(s, P, cand, active, best_ck, best_idx);
      g = 0;
      tile += tile_stride;
    }
  }

  if (MODE & kSelect)
    block_select_finish(best_ck, best_idx, P.sel, P.n_total, P.ib, s_ck, s_idx, P.gkey);
}

}  // namespace aceso
