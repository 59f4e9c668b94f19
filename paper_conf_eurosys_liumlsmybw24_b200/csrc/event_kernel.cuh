// event_kernel.cuh — event-driven evaluation of Aceso's performance/memory model (sm_100a).
//
// Same contract and outputs as eval_kernel.cuh (thread = candidate, warp = tile of 32,
// codes streamed through a per-warp cp.async.bulk ring), different arithmetic schedule:
//
// A stage's sums are sums over its RUNS (maximal op ranges of one (tp, dp) inside one
// stage). Within a run every op uses the same record key (b = mbs/dp, tp), so the run's
// contribution is a difference of position-prefix sums, PX[run][end] - PX[run][start],
// and its transient-memory term e is a range maximum (sparse table ST, two lookups).
// Recomputation only changes some ops of a run; its effect is the sum of per-op deltas
// (dS = fwd, dA = act - keep, dC = fwd_comp; e1 = peak + act - keep >= e0 = peak), looked
// up per 4-op quad and rc pattern from QR[signature][run][pattern].
//
// Phase A (lockstep over the code stream, 4 ops per step): per lane, one LOP3 finds the
// "events" of a quad (stage head, tp/dp change); a quad without events or recompute
// costs a handful of instructions and no table access. Events are appended to a per-lane
// list in shared memory; recompute deltas are accumulated in registers and, at a stage
// head, moved to a per-lane snapshot list (they belong to the stage the head closes).
// Phase B (drain, lockstep over list entries): every lane processes its k-th event at
// step k — the warp runs max_lane(#events) steps instead of one step per op position at
// which ANY lane has an event. An event closes the current run (prefix difference, range
// max; at a head also p2p_fwd, the snapshot, and the stage: Eq. 1/2, OOM, Heuristic-1)
// and opens the next (validity, p2p_bwd or reshard, prefix base). The lists drain when
// one could overflow and at the end of each tile.
//
// Paper: configuration (§3.1), Heuristic-1, memory Eq. 1
// (P:L225-234), time Eq. 2; readings R1-R13 in DESIGN.md §3.
#pragma once
#include "eval_kernel.cuh"

namespace aceso {

constexpr int kEvCap = 32;        // events per lane between drains (a chunk adds <= 16)
constexpr int kSnCap = 4;         // recompute snapshots per lane between drains (a quad adds <= 4)
constexpr int kEvRingSlots = 2;   // per-warp ring depth
constexpr int kEvSlotChunks = 4;  // 16-op chunks per ring slot (2 KB)
constexpr int kEvSlotBytes = kEvSlotChunks * 512;

__host__ __device__ constexpr uint32_t ev_ring_bytes() { return (uint32_t)kWarps * kEvRingSlots * kEvSlotBytes; }
__host__ __device__ constexpr uint32_t ev_list_bytes() { return (uint32_t)kWarps * kEvCap * 32 * 2; }
__host__ __device__ constexpr uint32_t ev_snap_bytes(bool full) {
  return (uint32_t)kWarps * kSnCap * 32 * (full ? 28u : 20u);
}

__device__ __forceinline__ uint64_t u64of(uint32_t lo, uint32_t hi) {
  return ((uint64_t)hi << 32) | lo;
}
__device__ __forceinline__ void sts32(uint32_t a, uint32_t v) {
  asm volatile("st.shared.u32 [%0], %1;" ::"r"(a), "r"(v) : "memory");
}
__device__ __forceinline__ void sts64(uint32_t a, uint64_t v) {
  asm volatile("st.shared.u64 [%0], %1;" ::"r"(a), "l"(v) : "memory");
}
__device__ __forceinline__ void sts16(uint32_t a, uint32_t v) {
  asm volatile("st.shared.u16 [%0], %1;" ::"r"(a), "h"((uint16_t)v) : "memory");
}
__device__ __forceinline__ uint64_t lds64u(uint32_t a) {
  uint64_t v;
  asm volatile("ld.shared.u64 %0, [%1];" : "=l"(v) : "r"(a));
  return v;
}

struct EvCand {
  // phase B: the open stage (prefix-difference form: -PX[start] + PX[end] per run)
  uint64_t S, A, W, D, comp;
  uint32_t E;
  uint32_t rr, dd, a;  // open run: (b, tp) index, (tp, dp) index, first op
  // phase A: recompute deltas since the last stage head
  uint64_t rS, rA, rC;
  uint32_t rE, rany;
  uint32_t cA;         // phase A: code of the last listed event (its run is the current one)
  uint32_t ec, sc, sp; // list entries, snapshots pushed, snapshots popped
  uint32_t sfl;        // bit k: list entry k (a single event, a head) takes the next snapshot
  // candidate-level aggregates (names shared with Cand: stage_commit / finish_cand)
  uint64_t sumS, bestT, bestM;
  uint32_t bt, bm, oom, i, gsum, reasons, nheads, head0, gst;
  uint32_t mbs, p, N;
};

// Dynamic shared memory: [qo][ring][event lists][snapshots S, A, (C), E]. The event list
// of a lane holds u16 entries (quad << 4 | mask of its events) at ev_base + 64 k; snapshot k of a lane
// is in per-field arrays (u64 S/A/C at +256 k, u32 E at +128 k).
struct EvSnap {
  uint32_t S, A, C, E;
};
// shared-memory address of the snapshot block (set once per CTA; read on the rare
// snapshot paths only, so the address does not occupy a register in the main loop)
__shared__ uint32_t ev_snap_base;
template <uint32_t MODE>
__device__ __forceinline__ EvSnap ev_snap_addr(uint32_t k) {
  const uint32_t lane = threadIdx.x & 31u, warp = threadIdx.x >> 5;
  const uint32_t snap = *(volatile uint32_t *)&ev_snap_base;
  const uint32_t blk64 = (uint32_t)kWarps * kSnCap * 256u;
  EvSnap a;
  a.S = snap + warp * kSnCap * 256u + lane * 8u + 256u * k;
  a.A = a.S + blk64;
  a.C = a.A + blk64;
  a.E = snap + ((MODE & kFull) ? 3u : 2u) * blk64 + warp * kSnCap * 128u + lane * 4u + 128u * k;
  return a;
}

__device__ __forceinline__ void ev_init(EvCand &s, const EvalParams &P, uint64_t h) {
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
  s.rr = s.dd = s.a = 0;
  s.rS = s.rA = s.rC = 0;
  s.rE = s.rany = 0;
  s.cA = 0;
  s.ec = s.sc = s.sp = 0;
  s.sfl = 0;
  s.sumS = s.bestT = s.bestM = 0;
  s.bt = s.bm = 0;
  s.oom = s.gsum = s.nheads = s.head0 = s.gst = 0;
  s.i = 0;
}

// (b, tp) run index of an op code under the candidate's mbs (clamped: invalid encodings
// still index inside the tables; their reasons are set when the run opens)
__device__ __forceinline__ uint32_t ev_run(uint32_t c, uint32_t mbs, const EvalParams &P) {
  const uint32_t tpl = (c >> 1) & 7u, dpl = c >> 5;
  const uint32_t b = min(dpl <= mbs ? mbs - dpl : 0u, (uint32_t)P.n_b - 1);
  return b * (uint32_t)P.n_tp + min(tpl, (uint32_t)P.n_tp - 1);
}

// recompute deltas of the ops of quad pattern pat (bit k = op 4q+k) under run rr
template <uint32_t MODE>
__device__ __forceinline__ void ev_rc_add(EvCand &s, const EvalParams &P, uint32_t qsb, uint32_t rr,
                                          uint32_t pat) {
  const uint32_t idx = qsb + rr * 16u + pat;
  const uint4 v0 = __ldg(P.qr + 2 * (size_t)idx);
  const uint4 v1 = __ldg(P.qr + 2 * (size_t)idx + 1);
  s.rS += u64of(v0.x, v0.y);
  s.rA += u64of(v0.z, v0.w);
  s.rE = max(s.rE, v1.x);
  if (MODE & kFull) s.rC += u64of(v1.z, v1.w);
  s.rany = 1u;
}

// 4-bit pattern of the bytes of a quad word whose bit `bit` is set (bits 0..3 = ops 0..3)
__device__ __forceinline__ uint32_t quad_bits(uint32_t v, int bit) {
  return ((((v >> bit) & 0x01010101u) * 0x01020408u) >> 24) & 0xfu;
}
// 4-bit pattern of the non-zero bytes of a quad word
__device__ __forceinline__ uint32_t quad_nonzero(uint32_t v) {
  const uint32_t y = (((v & 0x7f7f7f7fu) + 0x7f7f7f7fu) | v) & 0x80808080u;
  return quad_bits(y, 7);
}

// phase A, a quad of this lane with events and/or recompute flags (x = events, m = rc
// flags): recompute deltas are added per segment (ops between consecutive events share
// one run); each event is listed, a stage head first moving the deltas accumulated so
// far to a snapshot
template <uint32_t MODE>
__device__ __forceinline__ void ev_quad(EvCand &s, const EvalParams &P, uint32_t lev,
                                        uint32_t w, uint32_t x, uint32_t m, uint32_t qg,
                                        uint32_t qsb) {
  if (x == 0u) {  // recompute flags only: one pattern lookup under the current run
    ev_rc_add<MODE>(s, P, qsb, ev_run(s.cA, s.mbs, P), quad_bits(m, 4));
    return;
  }
  uint32_t evb = quad_nonzero(x);
  if (m == 0u && !(s.rany && (x & 0x01010101u))) {  // events only, no snapshot needed
    sts16(lev + 64u * s.ec, (qg << 4) | evb);  // one entry: the quad and its events
    s.ec += 1;
    s.cA = (w >> (8u * (31u - __clz(evb)))) & 0xffu;
    return;
  }
  const uint32_t pat = quad_bits(m, 4);
  evb |= 0x10u;  // + a virtual end of the quad at op 4
  uint32_t start = 0, cs = s.cA;
#pragma unroll 1
  while (true) {
    const uint32_t k = __ffs(evb) - 1u;
    evb &= evb - 1u;
    const uint32_t segp = pat & ((1u << k) - 1u) & ~((1u << start) - 1u);  // ops [start, k)
    if (segp) ev_rc_add<MODE>(s, P, qsb, ev_run(cs, s.mbs, P), segp);
    if (k == 4u) break;
    const uint32_t c = (w >> (8u * k)) & 0xffu;
    if ((c & 1u) && s.rany) {  // head: recompute deltas of the stage it closes
      const EvSnap a = ev_snap_addr<MODE>(s.sc);
      sts64(a.S, s.rS);
      sts64(a.A, s.rA);
      sts32(a.E, s.rE);
      if (MODE & kFull) sts64(a.C, s.rC);
      s.sc += 1;
      s.rS = s.rA = s.rC = 0;
      s.rE = 0;
      s.rany = 0;
      s.sfl |= 1u << s.ec;
    }
    sts16(lev + 64u * s.ec, (qg << 4) | (1u << k));
    s.ec += 1;
    cs = c;
    start = k;
  }
  s.cA = cs;
}

// activity word of a quad: bit 4 of a byte = recompute flag, other bits = event (head or
// tp/dp change against the previous op; p = the previous quad's word)
__device__ __forceinline__ uint32_t quad_activity(uint32_t w, uint32_t p) {
  const uint32_t sh = __funnelshift_l(p, w, 8);  // previous op's byte under each byte
  uint32_t d, f;
  asm("lop3.b32 %0, %1, %2, %3, 0xB4;" : "=r"(d) : "r"(w), "r"(sh), "r"(0x01010101u));  // c ? w : w^sh
  asm("lop3.b32 %0, %1, %2, %3, 0xD8;" : "=r"(f) : "r"(d), "r"(w), "r"(0x10101010u));   // c ? w : d
  return f;
}

// closes the open run [s.a, j) under s.rr (prefix difference, range max)
template <uint32_t MODE>
__device__ __forceinline__ void ev_close_run(EvCand &s, const EvalParams &P, uint32_t j) {
  const uint32_t Lp1 = (uint32_t)P.L + 1u;
  const size_t o = (size_t)s.rr * Lp1 + j;
  const uint4 x0 = __ldg(P.px + 2 * o);
  const uint4 x1 = __ldg(P.px + 2 * o + 1);
  const uint64_t dsum = __ldg(P.pd + (size_t)s.dd * Lp1 + j);
  const uint32_t k = 31u - __clz(j - s.a);
  const uint32_t *stk = P.st + ((size_t)k * P.runs + s.rr) * (uint32_t)P.L;
  const uint32_t e = max(__ldg(stk + s.a), __ldg(stk + j - (1u << k)));
  s.S += u64of(x0.x, x0.y);
  s.A += u64of(x0.z, x0.w);
  s.W += u64of(x1.x, x1.y);
  if (MODE & kFull) s.comp += u64of(x1.z, x1.w);
  s.D += dsum;
  s.E = max(s.E, e);
}

// phase B: one event (op j with code c opens a run; a head also closes a stage)
template <uint32_t MODE>
__device__ __forceinline__ void ev_handle(EvCand &s, const EvalParams &P, uint32_t j,
                                          uint32_t snapf, const unsigned char *cb, int64_t cand,
                                          bool active) {
  const uint32_t c = __ldg(cb + (j >> 4) * 512u + (j & 15u));  // the op's code (L2: just streamed)
  const uint32_t head = c & 1u;
  const uint32_t Lp1 = (uint32_t)P.L + 1u;
  const uint32_t *kx = reinterpret_cast<const uint32_t *>(P.kx);
  if (j > 0) {
    ev_close_run<MODE>(s, P, j);
    if (head) {
      s.S += __ldg(kx + 4 * ((size_t)s.rr * Lp1 + j) + 2);  // R5: p2p_fwd of the stage's last op
      if (snapf) {                                           // recompute deltas of this stage
        const EvSnap a = ev_snap_addr<MODE>(s.sp);
        s.S += lds64u(a.S);
        s.A -= lds64u(a.A);
        s.E = max(s.E, lds32(a.E));
        if (MODE & kFull) s.comp += lds64u(a.C);
        s.sp += 1;
      }
      stage_commit<MODE>(s, P, cand, active, false);
      s.i += 1;
    }
  }
  // open the run of op j: validity, table keys, p2p_bwd / reshard, prefix base
  const uint32_t tpl = (c >> 1) & 7u, dpl = c >> 5;
  if (dpl > s.mbs) s.reasons |= ACESO_R_DPMBS;
  if (tpl >= (uint32_t)P.n_tp || dpl >= (uint32_t)P.n_dp || (dpl <= s.mbs && s.mbs - dpl >= (uint32_t)P.n_b))
    s.reasons |= ACESO_R_TABLE;
  const uint32_t b = min(dpl <= s.mbs ? s.mbs - dpl : 0u, (uint32_t)P.n_b - 1);
  const uint32_t tplc = min(tpl, (uint32_t)P.n_tp - 1), dplc = min(dpl, (uint32_t)P.n_dp - 1);
  s.rr = b * (uint32_t)P.n_tp + tplc;
  s.dd = tplc * (uint32_t)P.n_dp + dplc;
  const size_t o = (size_t)s.rr * Lp1 + j;
  const uint32_t g = tpl + dpl;
  if (head || j == 0) {
    s.gst = g;
    s.gsum += 1u << g;  // R9
    s.nheads += head;
    if (head && j > 0) s.S += __ldg(kx + 4 * o + 1);  // R5: p2p_bwd of the first op
  } else {
    if (g != s.gst) s.reasons |= ACESO_R_GSTAGE;  // P:L151 in-stage symmetry
    s.S += __ldg(kx + 4 * o);                     // R13: reshard into this op
  }
  const uint4 y0 = __ldg(P.px + 2 * o);
  const uint4 y1 = __ldg(P.px + 2 * o + 1);
  s.S -= u64of(y0.x, y0.y);
  s.A -= u64of(y0.z, y0.w);
  s.W -= u64of(y1.x, y1.y);
  if (MODE & kFull) s.comp -= u64of(y1.z, y1.w);
  s.D -= __ldg(P.pd + (size_t)s.dd * Lp1 + j);
  s.a = j;
}

// phase B over every lane's list (warp-uniform call)
template <uint32_t MODE>
__device__ __forceinline__ void ev_drain(EvCand &s, const EvalParams &P, uint32_t lev,
                                         const unsigned char *cb, int64_t cand, bool active) {
  const uint32_t mx = __reduce_max_sync(0xffffffffu, s.ec);
#pragma unroll 1
  for (uint32_t k = 0; k < mx; ++k) {
    if (k < s.ec) {
      const uint32_t ent = lds16(lev + 64u * k);  // quad << 4 | event mask
      const uint32_t snapf = (s.sfl >> k) & 1u;
      uint32_t m = ent & 0xfu;
#pragma unroll 1
      do {
        const uint32_t b = __ffs(m) - 1u;
        m &= m - 1u;
        ev_handle<MODE>(s, P, (ent >> 4) * 4u + b, snapf, cb, cand, active);
      } while (m);
    }
  }
  s.ec = s.sc = s.sp = 0;
  s.sfl = 0;
}

// activity words of a chunk's 4 quads (w4 = its 16 code bytes, pw = the previous word)
struct ChunkAct {
  uint32_t f0, f1, f2, f3;
  __device__ __forceinline__ uint32_t get(uint32_t q) const {
    return q == 0u ? f0 : q == 1u ? f1 : q == 2u ? f2 : f3;
  }
};
__device__ __forceinline__ ChunkAct chunk_activity(uint4 w4, uint32_t pw) {
  return {quad_activity(w4.x, pw), quad_activity(w4.y, w4.x), quad_activity(w4.z, w4.y),
          quad_activity(w4.w, w4.z)};
}
__device__ __forceinline__ uint32_t word_of(uint4 w4, uint32_t q) {
  return q == 0u ? w4.x : q == 1u ? w4.y : q == 2u ? w4.z : w4.w;
}

// heads in a chunk (upper bound of the snapshots it can push)
__device__ __forceinline__ uint32_t chunk_heads(uint4 w4) {
  uint32_t h;
  asm("lop3.b32 %0, %1, %2, %3, 0xFE;" : "=r"(h) : "r"(w4.x & 0x01010101u), "r"((w4.y & 0x01010101u) << 1),
      "r"((w4.z & 0x01010101u) << 2));
  return __popc(h | ((w4.w & 0x01010101u) << 3));
}

// ops >= L of the last chunk (zero padding) take the last op's tp/dp without head or
// recompute: no events, no deltas (nvl = valid ops of the chunk, 1..15)
__device__ __forceinline__ uint4 pad_tail(uint4 w4, uint32_t nvl) {
  const uint32_t i = (nvl - 1u) >> 2;
  const uint32_t lw = i == 0u ? w4.x : i == 1u ? w4.y : i == 2u ? w4.z : w4.w;
  const uint32_t f = ((lw >> (8u * ((nvl - 1u) & 3u))) & 0xeeu) * 0x01010101u;
  auto keep = [&](uint32_t k) {  // valid-byte mask of word k
    return nvl >= 4u * k + 4u ? 0xffffffffu : nvl <= 4u * k ? 0u : (1u << (8u * (nvl - 4u * k))) - 1u;
  };
  uint32_t m;
  m = keep(0); w4.x = (w4.x & m) | (f & ~m);
  m = keep(1); w4.y = (w4.y & m) | (f & ~m);
  m = keep(2); w4.z = (w4.z & m) | (f & ~m);
  m = keep(3); w4.w = (w4.w & m) | (f & ~m);
  return w4;
}

template <uint32_t MODE, int MINB>
__global__ void __launch_bounds__(kThreads, MINB) event_kernel(const __grid_constant__ EvalParams P) {
  extern __shared__ __align__(128) unsigned char sm_raw[];
  __shared__ __align__(8) uint64_t s_tbar;
  __shared__ __align__(8) uint64_t s_ring_bar[kWarps][kEvRingSlots];
  __shared__ uint64_t s_ck[kWarps];
  __shared__ int64_t s_idx[kWarps];
  __shared__ unsigned int s_done;  // warps of this CTA past the tile loop

  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const uint32_t sb = smem_addr(sm_raw);
  // layout: [qo][ring][event lists][snapshots S, A, (C), E]
  const uint32_t qo = sb;
  const uint32_t ring = sb + P.qo_bytes + (uint32_t)warp * kEvRingSlots * kEvSlotBytes;
  const uint32_t lists = sb + P.qo_bytes + ev_ring_bytes();
  const uint32_t lev = lists + (uint32_t)warp * kEvCap * 64u + lane * 2u;  // this lane's event list
  if (threadIdx.x == 0) ev_snap_base = lists + ev_list_bytes();

  if (threadIdx.x == 0) {
    mbar_init(smem_addr(&s_tbar), 1);
    fence_barrier_init();
    s_done = 0;
  }
  if (lane == 0) {
    for (int k = 0; k < kEvRingSlots; ++k) mbar_init(smem_addr(&s_ring_bar[warp][k]), 1);
    fence_barrier_init();
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    const uint32_t bar = smem_addr(&s_tbar);
    mbar_expect_tx(bar, P.qo_bytes);
    bulk_g2s(qo, P.evblob + P.qo_off, P.qo_bytes, bar);
  }

  const uint32_t nch = (uint32_t)P.nch;
  const uint32_t ngroups = (nch + kEvSlotChunks - 1) / kEvSlotChunks;
  const int64_t first_tile = (int64_t)blockIdx.x * kWarps + warp;
  const int64_t tile_stride = (int64_t)gridDim.x * kWarps;
  const int64_t my_tiles =
      first_tile < P.n_tiles ? (P.n_tiles - first_tile + tile_stride - 1) / tile_stride : 0;
  const int64_t units = my_tiles * ngroups;
  const unsigned char *codes = reinterpret_cast<const unsigned char *>(P.codes);

  int64_t it_tile = first_tile;
  uint32_t it_g = 0;
  auto issue_next = [&](int slot) {
    const uint32_t a = kEvSlotChunks * it_g, b = min(a + kEvSlotChunks, nch);
    const uint32_t bar = smem_addr(&s_ring_bar[warp][slot]);
    mbar_expect_tx(bar, (b - a) * 512u);
    bulk_g2s(ring + slot * kEvSlotBytes, codes + ((size_t)it_tile * nch + a) * 512, (b - a) * 512u, bar);
    if (++it_g == ngroups) {
      it_g = 0;
      it_tile += tile_stride;
    }
  };
  if (lane == 0) {
    for (int64_t u = 0; u < units && u < kEvRingSlots; ++u) issue_next((int)u);
  }
  __syncwarp();
  mbar_wait(smem_addr(&s_tbar), 0);

  const uint32_t nvl = (uint32_t)P.L - 16u * (nch - 1u);  // valid ops of the last chunk
  const uint32_t ring_lane = ring + lane * 16u;
  const uint32_t bar0 = smem_addr(&s_ring_bar[warp][0]);

  uint64_t best_ck = ~0ull;
  int64_t best_idx = INT64_MAX;
  EvCand s;
  int slot = 0;
  uint32_t phase = 0;
  int64_t issued = kEvRingSlots;  // units issued so far (lane 0)
#pragma unroll 1
  for (int64_t tile = first_tile; tile < P.n_tiles; tile += tile_stride) {
    const int64_t cand = tile * 32 + lane;
    const bool active = cand < P.n;
    const unsigned char *cb = codes + (size_t)tile * nch * 512 + lane * 16;  // this lane's codes
    ev_init(s, P, active ? __ldg(P.hdr + cand) : 0ull);
    uint32_t pw = 0;
#pragma unroll 1
    for (uint32_t g = 0; g < ngroups; ++g) {
      mbar_wait(bar0 + 8u * slot, phase);
      const uint32_t ch0 = kEvSlotChunks * g, nc = min((uint32_t)kEvSlotChunks, nch - ch0);
      uint32_t addr = ring_lane + slot * kEvSlotBytes;
      if (g == 0) {
        // seed the previous word so that op 0 always shows a tp difference (an event)
        const uint32_t w0 = lds32(addr);
        pw = ((w0 & 0xffu) ^ 0x02u) << 24;
        s.head0 = w0 & 1u;
      }
      if (g == ngroups - 1u && nvl < 16u) {
        // ops >= L of the last chunk (zero padding) take the last op's tp/dp without head
        // or recompute: no events, no deltas (patched in this lane's ring copy)
        const uint32_t la = addr + (nc - 1u) * 512u;
        const uint4 t = pad_tail(lds128(la), nvl);
        asm volatile("st.shared.v4.u32 [%0], {%1, %2, %3, %4};" ::"r"(la), "r"(t.x), "r"(t.y), "r"(t.z),
                     "r"(t.w) : "memory");
      }
#pragma unroll 1
      for (uint32_t c = 0; c < nc; ++c, addr += 512u) {
        const uint32_t qg = (ch0 + c) * 4u;
        const uint4 w4 = lds128(addr);
        const ChunkAct fa = chunk_activity(w4, pw);
        pw = w4.w;
        const uint32_t lm = (fa.f0 ? 1u : 0u) | (fa.f1 ? 2u : 0u) | (fa.f2 ? 4u : 0u) | (fa.f3 ? 8u : 0u);
        // The lists must hold what the chunk adds (<= 16 events, <= its heads snapshots);
        // a chunk with more heads than snapshot slots in some lane goes quad by quad.
        const uint32_t h = chunk_heads(w4);
        const uint32_t rare = (h > (uint32_t)kSnCap ? 0x20u : 0u) |
                              ((s.ec + 16u > (uint32_t)kEvCap || s.sc + h > (uint32_t)kSnCap) ? 0x10u : 0u);
        const uint32_t v = __reduce_or_sync(0xffffffffu, lm | rare);
        if (v & 0x30u) {
          // rare path: drain first; quad by quad when careful
          uint32_t todo = v & 0xfu;
          const bool careful = (v & 0x20u) != 0u;
#pragma unroll 1
          do {
            const bool one = careful && todo != 0u;
            const uint32_t q = one ? __ffs(todo) - 1u : 0u;
            const uint32_t heads = one ? __popc(word_of(w4, q) & 0x01010101u) : h;
            const uint32_t evmax = one ? 4u : 16u;
            const bool full_soon = s.ec + evmax > (uint32_t)kEvCap || s.sc + heads > (uint32_t)kSnCap;
            if (__any_sync(0xffffffffu, full_soon)) ev_drain<MODE>(s, P, lev, cb, cand, active);
            const uint32_t now = one ? (1u << q) : todo;
#pragma unroll 1
            for (uint32_t t = now; t; t &= t - 1u) {
              const uint32_t qq = __ffs(t) - 1u;
              const uint32_t f = fa.get(qq);
              if (f)
                ev_quad<MODE>(s, P, lev, word_of(w4, qq), f & 0xefefefefu, f & 0x10101010u, qg + qq,
                              lds32(qo + 4u * (qg + qq)));
            }
            todo &= ~now;
          } while (todo);
        } else if (v) {
          if ((v & 1u) && fa.f0)
            ev_quad<MODE>(s, P, lev, w4.x, fa.f0 & 0xefefefefu, fa.f0 & 0x10101010u, qg, lds32(qo + 4u * qg));
          if ((v & 2u) && fa.f1)
            ev_quad<MODE>(s, P, lev, w4.y, fa.f1 & 0xefefefefu, fa.f1 & 0x10101010u, qg + 1u, lds32(qo + 4u * qg + 4u));
          if ((v & 4u) && fa.f2)
            ev_quad<MODE>(s, P, lev, w4.z, fa.f2 & 0xefefefefu, fa.f2 & 0x10101010u, qg + 2u, lds32(qo + 4u * qg + 8u));
          if ((v & 8u) && fa.f3)
            ev_quad<MODE>(s, P, lev, w4.w, fa.f3 & 0xefefefefu, fa.f3 & 0x10101010u, qg + 3u, lds32(qo + 4u * qg + 12u));
        }
      }
      __syncwarp();
      if (lane == 0 && issued < units) {
        fence_proxy_async();
        issue_next(slot);
        issued += 1;
      }
      if (++slot == kEvRingSlots) {
        slot = 0;
        phase ^= 1u;
      }
    }
    // ---- tile epilogue: drain, close the last run and stage (no p2p_fwd) ----
    ev_drain<MODE>(s, P, lev, cb, cand, active);
    ev_close_run<MODE>(s, P, (uint32_t)P.L);
    s.S += s.rS;
    s.A -= s.rA;
    s.E = max(s.E, s.rE);
    if (MODE & kFull) s.comp += s.rC;
    stage_commit<MODE>(s, P, cand, active, false);
    finish_cand<MODE>(s, P, cand, active, best_ck, best_idx);
  }

  if (MODE & kSelect) warp_select_finish(best_ck, best_idx, P.sel, P.n_total, P.ib, s_ck, s_idx, &s_done);
}

}  // namespace aceso
