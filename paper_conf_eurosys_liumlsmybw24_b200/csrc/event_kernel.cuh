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
// Phase A (lockstep over the code stream, one 16-op chunk per step): per lane, 3
// instructions per 4-op word give the chunk's ACTIVITY words (per op byte: bit 0 = stage
// head, bit 4 = recompute flag, bits 1-3 / 5-7 = tp / dp changed against the previous op).
// A chunk with events (head or tp/dp change) is appended to the lane's list (stores are
// unconditional, the count advances iff the chunk has events). A chunk with recompute
// flags but no events lies inside one run, so its recompute deltas are looked up right
// away (one pattern lookup per quad under the run of its ops) into per-lane CUMULATIVE
// sums; each list entry records the cumulative sums at its chunk and the recompute peak
// since the previous entry, so phase B attributes them to stages without snapshots.
// Phase B (drain, lockstep over ITEMS): every lane takes its next item in op order at
// each step — an event, or the recompute flags of one quad of an event chunk up to the
// quad's next event. The warp runs max_lane(#items) steps. An event closes the open run
// (prefix difference, range max; at a head also p2p_fwd, the phase-A recompute sums and
// the stage: Eq. 1/2, OOM, Heuristic-1) and opens the next (validity, p2p_bwd or reshard,
// prefix base). An event op's code is rebuilt from its activity byte and the open run's
// code (tp/dp bits are the XOR with the previous op, which belongs to the open run).
//
// Paper: configuration (§3.1), Heuristic-1, memory Eq. 1
// (P:L225-234), time Eq. 2; readings R1-R13 in DESIGN.md §3.
#pragma once
#include "eval_kernel.cuh"

namespace aceso {

constexpr int kEvCap = 4;         // event chunks per lane between drains (checked every 2 chunks)
constexpr int kEvRingSlots = 2;   // per-warp ring depth

// Dynamic shared memory: per warp one block of parts with lane stride 16 B (one per-lane base
// register lb = sb + ev_warp_bytes(SC) warp + 16 lane addresses them through immediate
// offsets, independent of the CTA's warp count W); SC = 16-op chunks per ring slot (4 or 8):
//   ring slot s  lb + 512 SC s + 512 c     the warp's cp.async.bulk ring (2 slots x SC chunks)
//   F            lb + ev_f_off(SC) + 512 k list entry k: activity words of the chunk
//   C            lb + ev_c_off(SC) + 512 k cumulative phase-A recompute sums dS, dA (u64 x 2)
// then X = [warp][k][lane] records {recompute peak since the previous entry, chunk index}
// (8 B; FULL: 16 B with the cumulative dC), addressed from lx = sb + ev_x_off(W, SC) + rec
// (warp, lane), and (SC = 4) the per-quad signature table (runtime size). With SC = 8 the
// signature table is read through the L1 (__ldg) instead, so two CTAs of 8 warps still fit.
static_assert(kEvCap * 512 == 2048, "per-warp list parts are 2 KB");
__host__ __device__ constexpr uint32_t ev_slot_bytes(int sc) { return 512u * (uint32_t)sc; }
__host__ __device__ constexpr uint32_t ev_f_off(int sc) { return 2u * ev_slot_bytes(sc); }
__host__ __device__ constexpr uint32_t ev_c_off(int sc) { return ev_f_off(sc) + 2048u; }
__host__ __device__ constexpr uint32_t ev_warp_bytes(int sc) { return ev_c_off(sc) + 2048u; }
__host__ __device__ constexpr uint32_t ev_xrec(bool full) { return full ? 16u : 8u; }
__host__ __device__ constexpr uint32_t ev_x_off(uint32_t w, int sc) { return w * ev_warp_bytes(sc); }
__host__ __device__ constexpr uint32_t ev_qo_off(bool full, uint32_t w, int sc) {
  return w * (ev_warp_bytes(sc) + kEvCap * 32u * ev_xrec(full));
}
// dynamic shared memory of one CTA (qo_bytes: the signature table's size)
__host__ __device__ constexpr uint32_t ev_smem_bytes(bool full, uint32_t w, int sc, uint32_t qo_bytes) {
  return ev_qo_off(full, w, sc) + (sc == 8 ? 0u : qo_bytes);
}

__device__ __forceinline__ uint64_t u64of(uint32_t lo, uint32_t hi) {
  return ((uint64_t)hi << 32) | lo;
}
__device__ __forceinline__ void sts64x2(uint32_t a, uint32_t x, uint32_t y) {
  asm volatile("st.shared.v2.u32 [%0], {%1, %2};" ::"r"(a), "r"(x), "r"(y) : "memory");
}
__device__ __forceinline__ uint2 lds64x2(uint32_t a) {
  uint2 v;
  asm volatile("ld.shared.v2.u32 {%0, %1}, [%2];" : "=r"(v.x), "=r"(v.y) : "r"(a));
  return v;
}
__device__ __forceinline__ uint32_t lds8(uint32_t a) {
  uint16_t v;
  asm volatile("ld.shared.u8 %0, [%1];" : "=h"(v) : "r"(a));
  return v;
}
__device__ __forceinline__ void sts128(uint32_t a, uint4 v) {
  asm volatile("st.shared.v4.u32 [%0], {%1, %2, %3, %4};" ::"r"(a), "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w)
               : "memory");
}

// Per-candidate state. Small fields are packed (registers are the occupancy limit):
//   run = rr | dd << 8 | cc << 16   open run: (b, tp) index (< 128), (tp, dp) index (< 64),
//                                   code of its first op (tp/dp bits = every op of the run)
//   fl  = bt | bm << 8 | oom << 16 | head0 << 17 | gst << 20
//         Heuristic-1 argmax stages (low 8 bits of the index; only valid candidates, whose
//         p <= 64, report them), any stage OOM, op 0 has a head, 2^gst devices in the open stage
//   hd  = mbs | p << 8              header: log2 microbatch, stage count
struct EvCand {
  // the open stage (prefix-difference form: -PX[start] + PX[end] per run)
  uint64_t S, A, W, D, comp;
  uint32_t E;
  uint32_t a;   // open run: first op
  uint32_t run;
  uint32_t ec;  // phase A: list entries
  // candidate-level aggregates
  uint64_t sumS, bestT, bestM;
  uint32_t i;   // stages closed so far (= heads at ops > 0)
  uint32_t gsum, reasons, N, fl, hd;
  __device__ __forceinline__ uint32_t rr() const { return run & 0xffu; }
  __device__ __forceinline__ uint32_t dd() const { return (run >> 8) & 0xffu; }
  __device__ __forceinline__ uint32_t cc() const { return run >> 16; }
  __device__ __forceinline__ uint32_t mbs() const { return hd & 0xffu; }
  __device__ __forceinline__ uint32_t p() const { return hd >> 8; }
};

__device__ __forceinline__ void ev_init(EvCand &s, const EvalParams &P, uint64_t h) {
  const uint32_t mbs = (uint32_t)(h & 0xff), p = (uint32_t)((h >> 8) & 0xff);
  s.hd = mbs | (p << 8);
  s.reasons = (h >> 16) ? ACESO_R_HDR : 0u;
  s.N = 0;
  if (mbs >= 62 || (1ull << mbs) > P.Bg || (P.Bg & ((1ull << mbs) - 1)) != 0)
    s.reasons |= ACESO_R_MBS;
  else
    s.N = (uint32_t)(P.Bg >> mbs);
  if (p == 0 || p > (uint32_t)P.G) s.reasons |= ACESO_R_PRANGE;
  s.S = s.A = s.W = s.D = s.comp = 0;
  s.E = 0;
  s.a = 0;
  s.run = 0;
  s.ec = 0;
  s.sumS = s.bestT = s.bestM = 0;
  s.fl = 0;
  s.gsum = 0;
  s.i = 0;
}

// Closes stage s.i: Eq. 2 key, Eq. 1 memory, OOM, Heuristic-1 maxima (ascending stage
// order, strict > keeps the lowest index on ties, R11), FULL per-stage outputs.
template <uint32_t MODE>
__device__ __forceinline__ void ev_commit(EvCand &s, const EvalParams &P, int64_t c, bool active) {
  s.sumS += s.S;
  const uint64_t tk = (uint64_t)(s.N - P.n_minus) * s.S + s.D;  // T_i - sum_k S_k (Eq. 2, R1, R6)
  const uint32_t p = s.p();
  const uint64_t infl = p > s.i ? (uint64_t)min(p - s.i, s.N) : 0ull;  // R2
  const uint64_t M = (s.W + infl * s.A + s.E) << P.mem_shift;         // Eq. 1 (R3, R4)
  const uint32_t i8 = s.i & 0xffu;
  if (tk > s.bestT) { s.bestT = tk; s.fl = (s.fl & ~0xffu) | i8; }
  if (M > s.bestM) { s.bestM = M; s.fl = (s.fl & ~0xff00u) | (i8 << 8); }
  if (M > P.C) s.fl |= 1u << 16;  // R10
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

// Candidate epilogue: validity, summary outputs, fused argmin (same contract as
// finish_cand of eval_kernel.cuh).
template <uint32_t MODE>
__device__ __forceinline__ void ev_finish(EvCand &s, const EvalParams &P, int64_t c, bool active,
                                          uint64_t &best_ck, int64_t &best_idx) {
  const uint32_t head0 = (s.fl >> 17) & 1u, p = s.p();
  uint32_t reasons = s.reasons;
  if (!head0) reasons |= ACESO_R_HEAD0;
  if (s.i + head0 != p) reasons |= ACESO_R_NSTAGE;  // heads = heads at ops > 0 + op 0's
  if (s.gsum != (uint32_t)P.G) reasons |= ACESO_R_GSUM;
  const bool invalid = reasons != 0;
  const bool oom = (s.fl >> 16) & 1u;
  const uint64_t iter = invalid ? 0ull : s.sumS + s.bestT;  // max_i T_i (Eq. 2)
  const uint64_t mem = invalid ? 0ull : s.bestM;
  uint32_t info = (p << 8);
  if (invalid) info |= ACESO_INFO_INVALID | (reasons << 18);
  else info |= (oom ? (((s.fl >> 8) & 0xffu) | ACESO_INFO_OOM) : (s.fl & 0xffu));  // Heuristic-1
  if (active) {
    if (MODE & kSummary) {
      P.iter_ns[c] = iter;
      P.max_mem[c] = mem;
      P.info[c] = info;
    }
    if ((MODE & kFull) && !invalid) {
      const uint32_t ns = min(p, (uint32_t)P.p_max);
      for (uint32_t k = 0; k < ns; ++k) P.stage_T[(int64_t)k * P.n + c] += s.sumS;
    }
    if ((MODE & kSelect) && !invalid) {
      // class 0 feasible (cost = iteration time), class 1 OOM (cost = max memory), R12
      const uint64_t ck = oom ? ((1ull << 62) | mem) : iter;
      const int64_t g = P.gofs + c;
      if (key_less(ck, g, best_ck, best_idx)) {
        best_ck = ck;
        best_idx = g;
      }
    }
  }
}

// recompute deltas of the ops of quad pattern pat (bit k = op 4q+k) under run rr
// (R3, R4, R7): dS = fwd, dA = act - keep, e1 = peak + act - keep, dC = fwd_comp
template <uint32_t MODE>
__device__ __forceinline__ void ev_rc_lookup(const EvalParams &P, uint32_t qsb, uint32_t rr, uint32_t pat,
                                             uint64_t &dS, uint64_t &dA, uint32_t &e1, uint64_t &dC) {
  const uint32_t idx = qsb + rr * 16u + pat;
  const uint4 v0 = __ldg(P.qr + 2u * idx);
  const uint4 v1 = __ldg(P.qr + 2u * idx + 1u);
  dS += u64of(v0.x, v0.y);
  dA += u64of(v0.z, v0.w);
  e1 = max(e1, v1.x);
  if (MODE & kFull) dC += u64of(v1.z, v1.w);
}
// the same for an octet pattern (bit k = op 8o+k) from the octet records (8-chunk slots)
template <uint32_t MODE>
__device__ __forceinline__ void ev_rc_lookup8(const EvalParams &P, uint32_t osb, uint32_t rr, uint32_t pat,
                                              uint64_t &dS, uint64_t &dA, uint32_t &e1, uint64_t &dC) {
  const uint32_t idx = osb + rr * 256u + pat;
  const uint4 v0 = __ldg(P.qr8 + 2u * idx);
  const uint4 v1 = __ldg(P.qr8 + 2u * idx + 1u);
  dS += u64of(v0.x, v0.y);
  dA += u64of(v0.z, v0.w);
  e1 = max(e1, v1.x);
  if (MODE & kFull) dC += u64of(v1.z, v1.w);
}
// phase B: recompute deltas of a quad pattern under the open run, into the open stage
template <uint32_t MODE>
__device__ __forceinline__ void ev_rc_add(EvCand &s, const EvalParams &P, uint32_t qsb, uint32_t pat,
                                          bool oct = false) {
  uint64_t dS = 0, dA = 0, dC = 0;
  uint32_t e1 = 0;
  if (oct)
    ev_rc_lookup8<MODE>(P, qsb, s.rr(), pat, dS, dA, e1, dC);
  else
    ev_rc_lookup<MODE>(P, qsb, s.rr(), pat, dS, dA, e1, dC);
  s.S += dS;
  s.A -= dA;
  s.E = max(s.E, e1);
  if (MODE & kFull) s.comp += dC;
}
// (b, tp) run index of an op code under the candidate's mbs (clamped exactly like
// ev_handle, so invalid encodings still index inside the tables)
__device__ __forceinline__ uint32_t ev_run(uint32_t c, uint32_t mbs, const EvalParams &P) {
  const uint32_t tpl = (c >> 1) & 7u, dpl = c >> 5;
  const uint32_t b = min(dpl <= mbs ? mbs - dpl : 0u, (uint32_t)P.n_b - 1);
  return b * (uint32_t)P.n_tp + min(tpl, (uint32_t)P.n_tp - 1);
}
// 4-bit pattern of the recompute flags (bit 4 of each byte) of a quad's activity word
__device__ __forceinline__ uint32_t quad_rc(uint32_t f) {
  return (((f & 0x10101010u) * 0x01020408u) >> 28);
}

// 8-bit pattern of the recompute flags of an octet (activity words a = ops 0-3, b = ops 4-7):
// one multiply gathers a's flags to bits 24-27 and b's to bits 28-31 (checked exhaustively:
// the cross terms fall below bit 24 or above bit 31)
__device__ __forceinline__ uint32_t octet_rc(uint32_t a, uint32_t b) {
  return ((((a & 0x10101010u) >> 4) | (b & 0x10101010u)) * 0x01020408u) >> 24;
}

// activity word of a quad: bit 4 of a byte = recompute flag, bit 0 = head, other bits =
// tp/dp change against the previous op (p = the previous quad's word)
__device__ __forceinline__ uint32_t quad_activity(uint32_t w, uint32_t p) {
  const uint32_t sh = __funnelshift_l(p, w, 8);  // previous op's byte under each byte
  uint32_t d, f;
  asm("lop3.b32 %0, %1, %2, %3, 0xB4;" : "=r"(d) : "r"(w), "r"(sh), "r"(0x01010101u));  // c ? w : w^sh
  asm("lop3.b32 %0, %1, %2, %3, 0xD8;" : "=r"(f) : "r"(d), "r"(w), "r"(0x10101010u));   // c ? w : d
  return f;
}

// closes the open run [s.a, j) under s.rr (prefix difference, range max); table offsets
// are 32-bit (the event tables are far below 4 G entries)
template <uint32_t MODE>
__device__ __forceinline__ void ev_close_run(EvCand &s, const EvalParams &P, uint32_t j) {
  const uint32_t Lp1 = (uint32_t)P.L + 1u;
  const uint32_t rr = s.rr();
  const uint32_t o = rr * Lp1 + j;
  const uint4 x0 = __ldg(P.px + 2u * o);
  const uint4 x1 = __ldg(P.px + 2u * o + 1u);
  const uint64_t dsum = __ldg(P.pd + (s.dd() * Lp1 + j));
  const uint32_t k = 31u - __clz(j - s.a);
  const uint32_t *stk = P.st + ((k * (uint32_t)P.runs + rr) * (uint32_t)P.L);
  const uint32_t e = max(__ldg(stk + s.a), __ldg(stk + (j - (1u << k))));
  s.S += u64of(x0.x, x0.y);
  s.A += u64of(x0.z, x0.w);
  s.W += u64of(x1.x, x1.y);
  if (MODE & kFull) s.comp += u64of(x1.z, x1.w);
  s.D += dsum;
  s.E = max(s.E, e);
}

// phase B: one event (op j with code c opens a run; a head also closes a stage)
// (cum, xad = shared-memory addresses of the entry's cumulative phase-A recompute sums
// dS, dA and dC)
template <uint32_t MODE>
__device__ __forceinline__ void ev_handle(EvCand &s, const EvalParams &P, uint32_t j, uint32_t c,
                                          uint32_t cum, uint32_t xad, int64_t cand, bool active) {
  const uint32_t head = c & 1u;
  const uint32_t Lp1 = (uint32_t)P.L + 1u;
  const uint32_t *kx = reinterpret_cast<const uint32_t *>(P.kx);
  if (j > 0) {
    ev_close_run<MODE>(s, P, j);
    if (head) {
      // phase-A recompute deltas: + cumulative sums at this chunk for the closing stage,
      // - the same for the opening one (prefix-difference form, exact mod 2^64)
      const uint4 cs = lds128(cum);
      const uint64_t cS = u64of(cs.x, cs.y), cA = u64of(cs.z, cs.w);
      uint64_t cC = 0;
      if (MODE & kFull) {
        const uint2 x = lds64x2(xad);
        cC = u64of(x.x, x.y);
      }
      s.S += __ldg(kx + (4u * (s.rr() * Lp1 + j) + 2u)) + cS;  // R5: p2p_fwd of the stage's last op
      s.A -= cA;
      if (MODE & kFull) s.comp += cC;
      ev_commit<MODE>(s, P, cand, active);
      s.i += 1;
      s.S -= cS;
      s.A += cA;
      if (MODE & kFull) s.comp -= cC;
    }
  }
  // open the run of op j: validity, table keys, p2p_bwd / reshard, prefix base
  const uint32_t tpl = (c >> 1) & 7u, dpl = c >> 5;
  const uint32_t mbs = s.mbs();
  if (dpl > mbs) s.reasons |= ACESO_R_DPMBS;
  if (tpl >= (uint32_t)P.n_tp || dpl >= (uint32_t)P.n_dp || (dpl <= mbs && mbs - dpl >= (uint32_t)P.n_b))
    s.reasons |= ACESO_R_TABLE;
  // clamped indices keep every gather inside the tables for invalid encodings
  const uint32_t b = min(dpl <= mbs ? mbs - dpl : 0u, (uint32_t)P.n_b - 1);
  const uint32_t tplc = min(tpl, (uint32_t)P.n_tp - 1), dplc = min(dpl, (uint32_t)P.n_dp - 1);
  const uint32_t rr = b * (uint32_t)P.n_tp + tplc;
  s.run = rr | ((tplc * (uint32_t)P.n_dp + dplc) << 8) | (c << 16);
  const uint32_t o = rr * Lp1 + j;
  const uint32_t g = tpl + dpl;
  if (head || j == 0) {
    s.fl = (s.fl & 0xfffffu) | (g << 20);
    s.gsum += 1u << g;  // R9
    if (head && j > 0) s.S += __ldg(kx + (4u * o + 1u));  // R5: p2p_bwd of the first op
  } else {
    if (g != (s.fl >> 20)) s.reasons |= ACESO_R_GSTAGE;  // P:L151 in-stage symmetry
    s.S += __ldg(kx + 4u * o);                     // R13: reshard into this op
  }
  const uint4 y0 = __ldg(P.px + 2u * o);
  const uint4 y1 = __ldg(P.px + 2u * o + 1u);
  s.S -= u64of(y0.x, y0.y);
  s.A -= u64of(y0.z, y0.w);
  s.W -= u64of(y1.x, y1.y);
  if (MODE & kFull) s.comp -= u64of(y1.z, y1.w);
  s.D -= __ldg(P.pd + (s.dd() * Lp1 + j));
  s.a = j;
}

// 16-bit masks of a chunk's activity words (bit k = op k of the chunk): ops with an event
// (any activity bit except the recompute bit 4) and ops with the recompute flag. Per word,
// one multiply gathers the 4 per-byte flag bits into bits 28-31 (no carries: every
// partial product lands on a distinct bit).
__device__ __forceinline__ uint32_t ev_nibble_hi(uint32_t w) {  // bit 7 of each byte -> bits 28..31
  return w * 0x00204081u;
}
__device__ __forceinline__ uint32_t ev_event_mask(uint4 f) {
  auto nz = [](uint32_t x) {  // bit 7 of each byte = byte & 0xef non-zero
    return ev_nibble_hi((((x & 0x6f6f6f6fu) + 0x7f7f7f7fu) | x) & 0x80808080u);
  };
  return (nz(f.x) >> 28) | ((nz(f.y) >> 24) & 0xf0u) | ((nz(f.z) >> 20) & 0xf00u) | ((nz(f.w) >> 16) & 0xf000u);
}
__device__ __forceinline__ uint32_t ev_rc_mask(uint4 f) {
  auto rc = [](uint32_t x) { return (x & 0x10101010u) * 0x01020408u; };  // bit 4 of byte b -> bit 28 + b
  return (rc(f.x) >> 28) | ((rc(f.y) >> 24) & 0xf0u) | ((rc(f.z) >> 20) & 0xf00u) | ((rc(f.w) >> 16) & 0xf000u);
}

// phase B over every lane's list (warp-uniform call), lockstep over ITEMS: each step every
// lane with work left takes its next item in op order — an event (run close/open, stage
// close) or a recompute segment (the recompute flags of one quad up to its next event:
// one pattern lookup under the open run). lb, lx = this lane's bases (see ev_warp_bytes).
template <uint32_t MODE, int SC, bool OCT>
__device__ __forceinline__ void ev_drain(EvCand &s, const EvalParams &P, uint32_t qo, uint32_t lb,
                                         uint32_t lx, int64_t cand, bool active) {
  constexpr uint32_t kEvF = ev_f_off(SC), kEvC = ev_c_off(SC);
  constexpr uint32_t XS = 32u * ev_xrec(MODE & kFull);  // X stride per entry
  uint32_t k = 0, em = 0, rm = 0, ent = 0, xe = 0, q0 = 0;
#pragma unroll 1
  while (true) {
    if ((em | rm) == 0u && k < s.ec) {  // next event chunk of this lane
      ent = lb + 512u * k;
      xe = lx + XS * k;
      const uint4 f4 = lds128(ent + kEvF);
      const uint2 ei = lds64x2(xe);
      s.E = max(s.E, ei.x);  // phase-A recompute peak since the previous entry (open stage)
      q0 = 4u * ei.y;
      em = ev_event_mask(f4);
      rm = ev_rc_mask(f4);
      ++k;
    }
    const uint32_t all = em | rm;
    if (!__any_sync(0xffffffffu, all != 0u)) break;
    if (all) {
      const uint32_t j = __ffs(all) - 1u;
      if ((em >> j) & 1u) {
        // the op's code: head and rc bits as stored, tp/dp = previous op's (the open run's) ^ change
        const uint32_t c = lds8(ent + kEvF + j) ^ (s.cc() & 0xeeu);
        ev_handle<MODE>(s, P, 4u * q0 + j, c, ent + kEvC, xe + 8u, cand, active);
        em &= em - 1u;
      } else {
        // recompute flags of quad j/4 (OCT: octet j/8) from op j up to its next event (all
        // bits of em and rm below j are consumed)
        const uint32_t qb = OCT ? (j & ~7u) : (j & ~3u);
        const uint32_t nxt = em & ((OCT ? 0xffu : 0xfu) << qb);
        const uint32_t lim = nxt ? __ffs(nxt) - 1u : qb + (OCT ? 8u : 4u);
        const uint32_t seg = rm & ((1u << lim) - 1u);
        uint32_t qsb;
        if (OCT)
          qsb = __ldg(P.qo8 + (q0 >> 1) + (j >> 3));  // q0 = 4 x chunk index
        else
          qsb = SC == 8 ? __ldg(reinterpret_cast<const uint32_t *>(P.evblob + P.qo_off) + (q0 + (j >> 2)))
                        : lds32(qo + 4u * (q0 + (j >> 2)));
        ev_rc_add<MODE>(s, P, qsb, seg >> qb, OCT);
        rm &= ~seg;
      }
    }
  }
  s.ec = 0;
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

// W warps per CTA (the launch uses 32 W threads), SC chunks per ring slot
// OCT: recompute-only chunks are looked up per octet (P.qr8, 2 lookups per chunk) instead of
// per quad (P.qr, 4 lookups); the quad tables still serve the drain's recompute items
template <uint32_t MODE, int MINB, int W, int SC, bool OCT>
__global__ void __launch_bounds__(32 * W, MINB) event_kernel(const __grid_constant__ EvalParams P) {
  constexpr uint32_t kEvSlotBytes = ev_slot_bytes(SC), kEvF = ev_f_off(SC), kEvC = ev_c_off(SC);
  constexpr bool QG = SC == 8;  // quad signature table read through the L1 (not staged)
  extern __shared__ __align__(128) unsigned char sm_raw[];
  __shared__ __align__(8) uint64_t s_tbar;
  __shared__ __align__(8) uint64_t s_ring_bar[kEvRingSlots][W];
  __shared__ uint64_t s_ck[W];
  __shared__ int64_t s_idx[W];
  constexpr bool FULL = (MODE & kFull) != 0;
  constexpr uint32_t XR = ev_xrec(FULL);

  const uint32_t lane = threadIdx.x & 31u, warp = threadIdx.x >> 5;
  const uint32_t sb = smem_addr(sm_raw);
  const uint32_t qo = sb + ev_qo_off(FULL, W, SC);
  const uint32_t lb = sb + warp * ev_warp_bytes(SC) + lane * 16u;  // see ev_warp_bytes
  const uint32_t lx = sb + ev_x_off(W, SC) + warp * kEvCap * 32u * XR + lane * XR;

  if (threadIdx.x == 0) {
    mbar_init(smem_addr(&s_tbar), 1);
    fence_barrier_init();
  }
  if (lane == 0) {
    for (int k = 0; k < kEvRingSlots; ++k) mbar_init(smem_addr(&s_ring_bar[k][warp]), 1);
    fence_barrier_init();
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    const uint32_t bar = smem_addr(&s_tbar);
    mbar_expect_tx(bar, QG ? 0u : P.qo_bytes);  // QG: the arrival alone completes the phase
    if (!QG) bulk_g2s(qo, P.evblob + P.qo_off, P.qo_bytes, bar);
  }

  const uint32_t nch = (uint32_t)P.nch;
  const uint32_t ngroups = (nch + SC - 1) / SC;
  // tile indices fit 32 bits (aceso_eval rejects n >= 2^37)
  const uint32_t n_tiles = (uint32_t)P.n_tiles;
  const uint32_t first_tile = blockIdx.x * W + warp;
  const uint32_t tile_stride = gridDim.x * W;
  const unsigned char *codes = reinterpret_cast<const unsigned char *>(P.codes);

  // producer state (lane 0): the next (tile, slot group) to copy; done when it_tile >= n_tiles
  uint32_t it_tile = first_tile;
  uint32_t it_g = 0;
  auto issue_next = [&](uint32_t slot) {
    const uint32_t a = SC * it_g, b = min(a + (uint32_t)SC, nch);
    const uint32_t bar = smem_addr(&s_ring_bar[slot][warp]);
    mbar_expect_tx(bar, (b - a) * 512u);
    bulk_g2s(lb + kEvSlotBytes * slot, codes + ((size_t)it_tile * nch + a) * 512, (b - a) * 512u, bar);
    if (++it_g == ngroups) {
      it_g = 0;
      it_tile += tile_stride;
    }
  };
  if (lane == 0) {
    for (uint32_t u = 0; u < (uint32_t)kEvRingSlots && it_tile < n_tiles; ++u) issue_next(u);
  }
  __syncwarp();
  mbar_wait(smem_addr(&s_tbar), 0);

  uint64_t best_ck = ~0ull;
  int64_t best_idx = INT64_MAX;
  EvCand s;
  ev_init(s, P, 0ull);
  uint64_t cS = 0, cA = 0, cC = 0;  // phase A: cumulative recompute deltas of the tile's event-free chunks
  uint32_t rE = 0;                  // phase A: their recompute peak since the last list entry
  uint32_t slot = 0, phase = 0;
  uint32_t pw = 0;       // phase A: the previous code word (its top byte = the previous op)
  int64_t cand = 0;
  bool active = false;
  // the lists must hold what the next 2 chunks add
  auto drain_check = [&]() {
    if (__any_sync(0xffffffffu, s.ec + 2u > (uint32_t)kEvCap)) ev_drain<MODE, SC, OCT>(s, P, qo, lb, lx, cand, active);
  };
  // phase A, one 16-op chunk (its 16 code bytes w4, chunk index ci)
  auto chunk = [&](const uint4 w4, uint32_t ci) {
    // OCT: the chunk's two octet signatures, requested ahead of the activity words (one
    // broadcast L1 load; its latency is off the recompute lookups' critical path)
    uint2 qsg = make_uint2(0u, 0u);
    if (OCT) asm volatile("ld.global.nc.v2.u32 {%0, %1}, [%2];"
                          : "=r"(qsg.x), "=r"(qsg.y) : "l"(P.qo8 + 2u * ci));
    uint4 f;
    f.x = quad_activity(w4.x, pw);
    f.y = quad_activity(w4.y, w4.x);
    f.z = quad_activity(w4.z, w4.y);
    f.w = quad_activity(w4.w, w4.z);
    pw = w4.w;
    const uint32_t orw = f.x | f.y | f.z | f.w;
    const bool evc = (orw & 0xefefefefu) != 0u;
    const bool rcc = !evc && (orw & 0x10101010u) != 0u;
    const uint32_t k = s.ec;
    const uint32_t e = lb + 512u * k;
    sts128(e + kEvF, f);
    sts128(e + kEvC, make_uint4((uint32_t)cS, (uint32_t)(cS >> 32), (uint32_t)cA, (uint32_t)(cA >> 32)));
    if (FULL)
      sts128(lx + 32u * XR * k, make_uint4(rE, ci, (uint32_t)cC, (uint32_t)(cC >> 32)));
    else
      sts64x2(lx + 32u * XR * k, rE, ci);
    if (evc) {
      rE = 0;
      s.ec = k + 1u;
    }
    if (__any_sync(0xffffffffu, rcc)) {
      if (rcc) {
        // recompute flags in an event-free chunk: every op is in the open run, whose
        // (tp, dp) is that of op 0 of the chunk
        const uint32_t rr = ev_run(w4.x & 0xffu, s.mbs(), P);
        if (OCT) {
          // two octet lookups (256-pattern records) instead of four quad lookups
          uint32_t pat;
          if ((pat = octet_rc(f.x, f.y))) ev_rc_lookup8<MODE>(P, qsg.x, rr, pat, cS, cA, rE, cC);
          if ((pat = octet_rc(f.z, f.w))) ev_rc_lookup8<MODE>(P, qsg.y, rr, pat, cS, cA, rE, cC);
        } else {
          const uint4 qs = QG ? __ldg(reinterpret_cast<const uint4 *>(P.evblob + P.qo_off) + ci)
                              : lds128(qo + 16u * ci);
          uint32_t pat;
          if ((pat = quad_rc(f.x))) ev_rc_lookup<MODE>(P, qs.x, rr, pat, cS, cA, rE, cC);
          if ((pat = quad_rc(f.y))) ev_rc_lookup<MODE>(P, qs.y, rr, pat, cS, cA, rE, cC);
          if ((pat = quad_rc(f.z))) ev_rc_lookup<MODE>(P, qs.z, rr, pat, cS, cA, rE, cC);
          if ((pat = quad_rc(f.w))) ev_rc_lookup<MODE>(P, qs.w, rr, pat, cS, cA, rE, cC);
        }
      }
    }
  };
#pragma unroll 1
  for (uint32_t tile = first_tile; tile < n_tiles; tile += tile_stride) {
    cand = (int64_t)tile * 32 + lane;
    active = cand < P.n;
    ev_init(s, P, active ? __ldg(P.hdr + cand) : 0ull);
    cS = cA = cC = 0;
    rE = 0;
    {
      // the tile's first slot: seed the previous word so that op 0 always shows a tp
      // difference (an event); the group loop's wait on this slot then returns at once
      mbar_wait(smem_addr(&s_ring_bar[0][warp]) + 8u * W * slot, phase);
      const uint32_t w0 = lds32(lb + kEvSlotBytes * slot);
      pw = ((w0 & 0xffu) ^ 0x02u) << 24;
      s.run = ((w0 & 0xffu) ^ 0x02u) << 16;  // phase B rebuilds op 0's code against the same seed
      s.fl = (w0 & 1u) << 17;                 // head0
    }
#pragma unroll 1
    for (uint32_t g = 0; g < ngroups; ++g) {
      const uint32_t ch0 = SC * g, nc = min((uint32_t)SC, nch - ch0);
      const uint32_t addr = lb + kEvSlotBytes * slot;
      mbar_wait(smem_addr(&s_ring_bar[0][warp]) + 8u * W * slot, phase);
      if (g == ngroups - 1u) {
        const uint32_t nvl = (uint32_t)P.L - 16u * (nch - 1u);  // valid ops of the last chunk
        if (nvl < 16u) {
          // ops >= L of the last chunk (zero padding) take the last op's tp/dp without head
          // or recompute: no events, no deltas (patched in this lane's ring copy)
          const uint32_t la = addr + (nc - 1u) * 512u;
          sts128(la, pad_tail(lds128(la), nvl));
        }
      }
      if (nc == (uint32_t)SC) {
#pragma unroll 1
        for (uint32_t h = 0; h < (uint32_t)SC; h += 4u) {
          // two chunks' code words requested back to back (the second chunk's shared-memory
          // latency hides behind the first chunk's work)
          drain_check();
          if (FULL) {  // (FULL modes: no paired loads; their extra live registers spill at 80)
            chunk(lds128(addr + 512u * h), ch0 + h);
            chunk(lds128(addr + 512u * h + 512u), ch0 + h + 1u);
          } else {
            const uint4 wa = lds128(addr + 512u * h), wb = lds128(addr + 512u * h + 512u);
            chunk(wa, ch0 + h);
            chunk(wb, ch0 + h + 1u);
          }
          drain_check();
          if (FULL) {
            chunk(lds128(addr + 512u * h + 1024u), ch0 + h + 2u);
            chunk(lds128(addr + 512u * h + 1536u), ch0 + h + 3u);
          } else {
            const uint4 wc = lds128(addr + 512u * h + 1024u), wd = lds128(addr + 512u * h + 1536u);
            chunk(wc, ch0 + h + 2u);
            chunk(wd, ch0 + h + 3u);
          }
        }
      } else {
#pragma unroll 1
        for (uint32_t c = 0; c < nc; ++c) {
          if ((c & 1u) == 0u) drain_check();
          chunk(lds128(addr + 512u * c), ch0 + c);
        }
      }
      __syncwarp();
      if (lane == 0 && it_tile < n_tiles) {
        fence_proxy_async();
        issue_next(slot);
      }
      slot ^= 1u;
      phase ^= slot ^ 1u;  // flips after slot 1
    }
    // ---- tile epilogue: drain, close the last run and stage (no p2p_fwd) ----
    ev_drain<MODE, SC, OCT>(s, P, qo, lb, lx, cand, active);
    s.S += cS;  // phase-A recompute deltas after the last event chunk (last stage)
    s.A -= cA;
    s.E = max(s.E, rE);
    if (MODE & kFull) s.comp += cC;
    ev_close_run<MODE>(s, P, (uint32_t)P.L);
    ev_commit<MODE>(s, P, cand, active);
    ev_finish<MODE>(s, P, cand, active, best_ck, best_idx);
  }

  if (MODE & kSelect) warp_select_finish(best_ck, best_idx, P.sel, P.n_total, P.ib, s_ck, s_idx, P.gkey);
}

}  // namespace aceso
