// scan_kernel.cuh — streaming evaluation of Aceso's performance/memory model (sm_100a).
//
// The default schedule of aceso_eval. Same contract and outputs as the other kernels
// (thread = candidate, warp = tile of 32 candidates in the tiled layout of include/aceso.h),
// exact in unsigned 64-bit arithmetic for every field width the header admits (memory
// values are not packed into 32-bit units).
//
// A stage's sums are sums over its RUNS (maximal op ranges of one (tp, dp) inside one stage;
// every op of a run reads its record under the same key (b = mbs/dp, tp), R8), so a run's
// contribution is a difference of position prefixes PX[key][end] - PX[key][start], its DP
// sync a difference of PD[(tp, dp)], and its transient-memory term a range maximum (sparse
// table). Recomputed ops add per-op deltas (P:L241 / R7: + forward; R3: act -> keep; R4:
// transient peak + act - keep), looked up per 4-op quad and recompute pattern.
//
// Work per tile (one warp):
//   scan   — the warp's tiles are one contiguous byte range of the batch, streamed through
//            a per-warp ring of 2 KB cp.async.bulk copies (mbarrier completion). Per 16-op
//            chunk a lane does one LDS.128 and tests whether all 16 codes equal the open
//            run's code with no head and no recompute flag ("clean", 3 LOP3 + 1 compare);
//            the chunk is appended to the lane's list unconditionally and the list grows
//            only for a dirty chunk.
//   drain  — when a list could overflow and at the end of the tile, every lane walks its
//            dirty chunks in op order (lockstep over ITEMS): an event (stage head or tp/dp
//            change: close the open run, at a head close the stage — Eq. 2, Eq. 1, OOM,
//            Heuristic-1 — open the next run), or the recompute flags of a quad segment
//            (one lookup); recompute flags after a chunk's last event all lie in the open
//            run and are resolved in one step (up to 4 lookups in flight).
//   finish — last run and stage, validity reasons, SoA outputs, fused argmin (warp, CTA,
//            last CTA of the grid).
//
// Paper: configuration (§3.1), Heuristic-1, Eq. 1,
// Eq. 2; readings R1-R13, R18-R20 in DESIGN.md §3.
#pragma once
#include <type_traits>

#include "eval_kernel.cuh"   // PTX helpers (mbarrier, cp.async.bulk, shared loads), mode bits
#include "event_kernel.cuh"  // activity words, event / recompute masks, pad_tail, u64of, lds8

namespace aceso {

constexpr uint32_t kScSlotChunks = 8;                       // chunks per bulk copy (4 KB)
constexpr uint32_t kScSlots = 2;                            // ring depth per warp
constexpr uint32_t kScCap = 6;                              // list entries per lane
constexpr uint32_t kScRingW = kScSlots * kScSlotChunks * 512u;
constexpr uint32_t kScListW = kScCap * 512u;                // [k][lane] 16 B: the chunk's codes
constexpr uint32_t kScMetaW = kScCap * 128u;                // [k][lane] 4 B: chunk << 8 | previous op
constexpr uint32_t kScMaskW = kScCap * 128u;                // [k][lane] 4 B: event mask | recompute mask << 16
constexpr uint32_t kScWarpBytes = kScRingW + kScListW + kScMetaW + kScMaskW;
__host__ __device__ constexpr uint32_t sc_smem_bytes(uint32_t qo_bytes) {
  return (uint32_t)kWarps * kScWarpBytes + qo_bytes;
}

__device__ __forceinline__ void sts32(uint32_t a, uint32_t v) {
  asm volatile("st.shared.u32 [%0], %1;" ::"r"(a), "r"(v) : "memory");
}

template <bool E64>
struct ScCand {
  using ET = typename std::conditional<E64, uint64_t, uint32_t>::type;
  // the open stage (prefix-difference form: -PX[start] + PX[end] per run)
  uint64_t S, A, W, D, C;
  ET E;          // transient-memory maximum, units of 2^es bytes
  uint32_t a;    // open run: first op
  uint32_t run;  // rr | dd << 8 | (code & 0xee) << 16: (b, tp) index, (tp, dp) index, tp/dp bits
  // candidate
  uint64_t sumS, bestT, bestM;
  uint32_t i;    // stages closed so far
  uint32_t gsum, reasons, N, fl, hd;  // fl: argmax T | argmax Mem << 8 | OOM << 16 | head0 << 17 | g << 20
  __device__ __forceinline__ uint32_t rr() const { return run & 0xffu; }
  __device__ __forceinline__ uint32_t dd() const { return (run >> 8) & 0xffu; }
  __device__ __forceinline__ uint32_t mbs() const { return hd & 0xffu; }
  __device__ __forceinline__ uint32_t p() const { return hd >> 8; }
};

template <bool E64>
__device__ __forceinline__ void sc_init(ScCand<E64> &s, const EvalParams &P, uint64_t h) {
  const uint32_t mbs = (uint32_t)(h & 0xff), p = (uint32_t)((h >> 8) & 0xff);
  s.hd = mbs | (p << 8);
  s.reasons = (h >> 16) ? ACESO_R_HDR : 0u;
  s.N = 0;
  if (mbs >= 62 || (1ull << mbs) > P.Bg || (P.Bg & ((1ull << mbs) - 1)) != 0)
    s.reasons |= ACESO_R_MBS;
  else
    s.N = (uint32_t)(P.Bg >> mbs);  // R8: N = Bg / mbs
  if (p == 0 || p > (uint32_t)P.G) s.reasons |= ACESO_R_PRANGE;
  s.S = s.A = s.W = s.D = s.C = 0;
  s.E = 0;
  s.a = 0;
  s.run = 0;
  s.sumS = s.bestT = s.bestM = 0;
  s.fl = 0;
  s.gsum = 0;
  s.i = 0;
}

// Closes stage s.i: Eq. 2 key (N-1) S_i + D_i (T_i minus the common sum, R1, R6), Eq. 1
// memory Wst + min(p-i, N) A + E (R2-R4), OOM (R10), Heuristic-1 maxima in ascending stage
// order (strict >: lowest index on ties, R11), FULL per-stage outputs.
template <uint32_t MODE, bool E64>
__device__ __forceinline__ void sc_commit(ScCand<E64> &s, const EvalParams &P, int64_t c, bool active) {
  s.sumS += s.S;
  const uint64_t tk = (uint64_t)(s.N - P.n_minus) * s.S + s.D;
  const uint32_t p = s.p();
  const uint64_t infl = p > s.i ? (uint64_t)min(p - s.i, s.N) : 0ull;
  const uint64_t M = s.W + infl * s.A + ((uint64_t)s.E << P.es);
  const uint32_t i8 = s.i & 0xffu;
  if (tk > s.bestT) { s.bestT = tk; s.fl = (s.fl & ~0xffu) | i8; }
  if (M > s.bestM) { s.bestM = M; s.fl = (s.fl & ~0xff00u) | (i8 << 8); }
  if (M > P.C) s.fl |= 1u << 16;
  if (MODE & kFull) {
    if (active && s.i < (uint32_t)P.p_max) {
      const int64_t o = (int64_t)s.i * P.n + c;
      P.stage_T[o] = tk;  // + sum_k S_k in sc_finish
      P.stage_mem[o] = M;
      P.stage_comp[o] = (uint64_t)s.N * s.C;
      P.stage_comm[o] = (uint64_t)s.N * (s.S - s.C) + s.D;
    }
  }
  s.S = s.A = s.W = s.D = s.C = 0;
  s.E = 0;
}

template <uint32_t MODE, bool E64>
__device__ __forceinline__ void sc_finish(ScCand<E64> &s, const EvalParams &P, int64_t c, bool active,
                                          uint64_t &best_ck, int64_t &best_idx) {
  const uint32_t head0 = (s.fl >> 17) & 1u, p = s.p();
  uint32_t reasons = s.reasons;
  if (!head0) reasons |= ACESO_R_HEAD0;
  if (s.i + head0 != p) reasons |= ACESO_R_NSTAGE;
  if (s.gsum != (uint32_t)P.G) reasons |= ACESO_R_GSUM;  // R9
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
      const uint64_t ck = oom ? ((1ull << 62) | mem) : iter;  // class 0 feasible, 1 OOM (R12)
      const int64_t g = P.gofs + c;
      if (key_less(ck, g, best_ck, best_idx)) {
        best_ck = ck;
        best_idx = g;
      }
    }
  }
}

// (b, tp) run key of an op code under the candidate's mbs, clamped into the tables (invalid
// encodings still index inside them; their outputs are suppressed)
__device__ __forceinline__ uint32_t sc_rr(uint32_t c, uint32_t mbs, const EvalParams &P) {
  const uint32_t tpl = (c >> 1) & 7u, dpl = c >> 5;
  const uint32_t b = min(dpl <= mbs ? mbs - dpl : 0u, (uint32_t)P.n_b - 1);
  return b * (uint32_t)P.n_tp + min(tpl, (uint32_t)P.n_tp - 1);
}

// recompute deltas of quad pattern `pat` at record base `qb` (signature offset) under run rr:
// S += forward (R7), A -= act - keep (R3), E = max(E, peak + act - keep) (R4), C += fwd_comp
template <uint32_t MODE, bool E64>
__device__ __forceinline__ void sc_rc(ScCand<E64> &s, const EvalParams &P, uint32_t qb, uint32_t rr,
                                      uint32_t pat) {
  const uint32_t idx = qb + rr * 16u + pat;
  const uint4 v0 = __ldg(P.sq + 2u * idx);
  const uint4 v1 = __ldg(P.sq + 2u * idx + 1u);
  s.S += u64of(v0.x, v0.y);
  s.A -= u64of(v0.z, v0.w);
  if (E64) s.E = max((uint64_t)s.E, u64of(v1.x, v1.y));
  else s.E = max((uint32_t)s.E, v1.x);
  if (MODE & kFull) s.C += u64of(v1.z, v1.w);
}

// closes the open run [s.a, j) under its keys: prefix differences and the range maximum
template <uint32_t MODE, bool E64>
__device__ __forceinline__ void sc_close_run(ScCand<E64> &s, const EvalParams &P, uint32_t j) {
  using ET = typename ScCand<E64>::ET;
  const uint32_t Lp1 = (uint32_t)P.L + 1u;
  const uint32_t rr = s.rr();
  const uint32_t o = rr * Lp1 + j;
  const uint4 x0 = __ldg(P.sx + 2u * o);
  const uint64_t pw = __ldg(reinterpret_cast<const unsigned long long *>(P.sx + 2u * o + 1u));
  const uint64_t dsum = __ldg(P.sd + (s.dd() * Lp1 + j));
  const uint32_t k = 31u - __clz(j - s.a);
  const ET *stk = reinterpret_cast<const ET *>(P.ss) + ((size_t)(k * (uint32_t)P.runs + rr) * (uint32_t)P.L);
  const ET e = max(__ldg(stk + s.a), __ldg(stk + (j - (1u << k))));
  s.S += u64of(x0.x, x0.y);
  s.A += u64of(x0.z, x0.w);
  s.W += pw;
  if (MODE & kFull) s.C += __ldg(reinterpret_cast<const unsigned long long *>(P.sx + 2u * o + 1u) + 1);
  s.D += dsum;
  s.E = max(s.E, e);
}

// one event: op j with code c opens a run (tp/dp change or stage head); a head at j > 0
// also closes the stage
template <uint32_t MODE, bool E64>
__device__ __forceinline__ void sc_event(ScCand<E64> &s, const EvalParams &P, uint32_t j, uint32_t c,
                                         int64_t cand, bool active) {
  const uint32_t head = c & 1u;
  const uint32_t Lp1 = (uint32_t)P.L + 1u;
  const uint32_t *kx = reinterpret_cast<const uint32_t *>(P.sk);
  if (j > 0) {
    sc_close_run<MODE, E64>(s, P, j);
    if (head) {
      s.S += __ldg(kx + (4u * (s.rr() * Lp1 + j) + 2u));  // R5: p2p_fwd of the stage's last op
      sc_commit<MODE, E64>(s, P, cand, active);
      s.i += 1;
    }
  }
  // open the run of op j: validity (R18), keys, p2p_bwd / reshard, prefix base
  const uint32_t tpl = (c >> 1) & 7u, dpl = c >> 5;
  const uint32_t mbs = s.mbs();
  if (dpl > mbs) s.reasons |= ACESO_R_DPMBS;
  if (tpl >= (uint32_t)P.n_tp || dpl >= (uint32_t)P.n_dp || (dpl <= mbs && mbs - dpl >= (uint32_t)P.n_b))
    s.reasons |= ACESO_R_TABLE;
  const uint32_t b = min(dpl <= mbs ? mbs - dpl : 0u, (uint32_t)P.n_b - 1);
  const uint32_t tplc = min(tpl, (uint32_t)P.n_tp - 1), dplc = min(dpl, (uint32_t)P.n_dp - 1);
  const uint32_t rr = b * (uint32_t)P.n_tp + tplc;
  const uint32_t dd = tplc * (uint32_t)P.n_dp + dplc;
  s.run = rr | (dd << 8) | ((c & 0xeeu) << 16);
  const uint32_t g = tpl + dpl;
  if (j == 0) {  // op 0 opens stage 0 (R19); every prefix is 0 at position 0
    s.fl = (s.fl & 0xfffffu) | (g << 20) | (head << 17);
    s.gsum += 1u << g;  // R9
    s.a = 0;
    return;
  }
  const uint32_t o = rr * Lp1 + j;
  if (head) {
    s.fl = (s.fl & 0xfffffu) | (g << 20);
    s.gsum += 1u << g;                              // R9
    s.S += __ldg(kx + (4u * o + 1u));               // R5: p2p_bwd of the stage's first op
  } else {
    if (g != (s.fl >> 20)) s.reasons |= ACESO_R_GSTAGE;  // P:L151 in-stage symmetry
    s.S += __ldg(kx + 4u * o);                            // R13: reshard into op j
  }
  const uint4 y0 = __ldg(P.sx + 2u * o);
  const uint64_t yw = __ldg(reinterpret_cast<const unsigned long long *>(P.sx + 2u * o + 1u));
  s.S -= u64of(y0.x, y0.y);
  s.A -= u64of(y0.z, y0.w);
  s.W -= yw;
  if (MODE & kFull) s.C -= __ldg(reinterpret_cast<const unsigned long long *>(P.sx + 2u * o + 1u) + 1);
  s.D -= __ldg(P.sd + (dd * Lp1 + j));
  s.a = j;
}

// event and recompute masks of a list entry (bit k = op 16 ch + k): events are stage heads and
// tp/dp changes against the previous op (op 0 always opens a segment, R19)
__device__ __forceinline__ void sc_masks(uint4 w, uint32_t m0, uint32_t &em, uint32_t &rm) {
  uint4 f;
  f.x = quad_activity(w.x, m0 << 24);  // previous op = the last op before the chunk
  f.y = quad_activity(w.y, w.x);
  f.z = quad_activity(w.z, w.y);
  f.w = quad_activity(w.w, w.z);
  em = ev_event_mask(f) | (((m0 >> 8) & 0x3ffu) == 0u ? 1u : 0u);
  rm = ev_rc_mask(f);
}

// list entry meta word: chunk << 8 | previous op's tp/dp code | recompute-only << 31 |
// resolved << 30 (a resolved entry holds {dS, dA} in its code slot and e1 in its mask word)
constexpr uint32_t kScRcOnly = 1u << 31, kScResolved = 1u << 30;

// Drain of the lists (warp-uniform call).
// (1) SUMMARY mode: the recompute-only chunks of all lanes (no head, no tp/dp change: every op
//     in the open run) are resolved at full SIMT width, one entry per thread: up to 4 quad
//     lookups, the deltas replace the entry's codes.
// (2) every lane walks its own entries in op order, event-synchronous: each step a lane
//     consumes its cheap items (resolved chunks, recompute segments) up to its next event,
//     then all lanes with one handle it together.
template <uint32_t MODE, bool E64>
__device__ __forceinline__ void sc_drain(ScCand<E64> &s, const EvalParams &P, uint32_t &cnt, uint32_t wl,
                                         uint32_t lane, uint32_t qo, int64_t cand, bool active) {
  constexpr bool RESOLVE = !E64 && !(MODE & kFull);
  const uint32_t wm0 = wl + kScListW, wm1 = wm0 + kScMetaW;  // warp bases of the meta / e1 arrays
  if (RESOLVE && P.sc_resolve) {
    __syncwarp();  // the lanes' list writes are visible to the compacted pass
    uint32_t incl = cnt;
#pragma unroll
    for (uint32_t o = 1; o < 32; o <<= 1) {
      const uint32_t v = __shfl_up_sync(0xffffffffu, incl, o);
      if (lane >= o) incl += v;
    }
    const uint32_t total = __shfl_sync(0xffffffffu, incl, 31);
    const uint32_t excl = incl - cnt, mymbs = s.mbs();
#pragma unroll 1
    for (uint32_t g0 = 0; g0 < total; g0 += 32) {
      const uint32_t g = g0 + lane;
      uint32_t l = 0;  // owner: the first lane whose inclusive count exceeds g
#pragma unroll
      for (uint32_t st = 16; st > 0; st >>= 1) {
        const uint32_t v = __shfl_sync(0xffffffffu, incl, l + st - 1u);
        if (v <= g) l += st;
      }
      const uint32_t k = g - __shfl_sync(0xffffffffu, excl, l);
      const uint32_t mbs = __shfl_sync(0xffffffffu, mymbs, l);
      const uint32_t m0a = wm0 + 128u * k + 4u * l;
      const uint32_t m0 = g < total ? lds32(m0a) : 0u;
      if (m0 & kScRcOnly) {
        const uint32_t slot = wl + 512u * k + 16u * l;
        const uint4 w = lds128(slot);
        const uint32_t rr = sc_rr(m0 & 0xffu, mbs, P);
        const uint4 qs = lds128(qo + 16u * ((m0 >> 8) & 0x3ffu));
        const uint32_t rw[4] = {w.x, w.y, w.z, w.w}, qb[4] = {qs.x, qs.y, qs.z, qs.w};
        uint64_t dS = 0, dA = 0;
        uint32_t e1 = 0;
#pragma unroll
        for (uint32_t q = 0; q < 4; ++q) {
          const uint32_t pat = quad_rc(rw[q]);
          if (pat) {
            const uint32_t idx = qb[q] + rr * 16u + pat;
            const uint4 v0 = __ldg(P.sq + 2u * idx);
            const uint32_t v1 = __ldg(reinterpret_cast<const uint32_t *>(P.sq + 2u * idx + 1u));
            dS += u64of(v0.x, v0.y);
            dA += u64of(v0.z, v0.w);
            e1 = max(e1, v1);
          }
        }
        sts128(slot, make_uint4((uint32_t)dS, (uint32_t)(dS >> 32), (uint32_t)dA, (uint32_t)(dA >> 32)));
        sts32(wm1 + 128u * k + 4u * l, e1);
        sts32(m0a, m0 | kScResolved);
      }
    }
    __syncwarp();
  }
  // ---- (2) per-lane walk ----
  const uint32_t lst = wl + 16u * lane, m0b = wm0 + 4u * lane, m1b = wm1 + 4u * lane;
  uint32_t k = 0, em = 0, rm = 0, ent = 0, ch = 0;
#pragma unroll 1
  while (true) {
    bool ev = false;
#pragma unroll 1
    while (true) {  // this lane's cheap items up to its next event
      if ((em | rm) == 0u) {
        if (k >= cnt) break;
        const uint32_t m0 = lds32(m0b + 128u * k);
        if (RESOLVE && (m0 & kScResolved)) {  // a resolved recompute-only chunk: into the open stage
          const uint4 v = lds128(lst + 512u * k);
          const uint32_t e1 = lds32(m1b + 128u * k);
          s.S += u64of(v.x, v.y);
          s.A -= u64of(v.z, v.w);
          s.E = max(s.E, (typename ScCand<E64>::ET)e1);
          ++k;
          continue;
        }
        ent = lst + 512u * k;
        ch = (m0 >> 8) & 0x3ffu;
        sc_masks(lds128(ent), m0, em, rm);
        ++k;
      }
      if (em == 0u) {
        // no event left in this chunk: its recompute flags lie in the open run
        const uint4 qs = lds128(qo + 16u * ch);
        const uint32_t rr = s.rr();
        uint32_t pat;
        if ((pat = rm & 0xfu)) sc_rc<MODE, E64>(s, P, qs.x, rr, pat);
        if ((pat = (rm >> 4) & 0xfu)) sc_rc<MODE, E64>(s, P, qs.y, rr, pat);
        if ((pat = (rm >> 8) & 0xfu)) sc_rc<MODE, E64>(s, P, qs.z, rr, pat);
        if ((pat = rm >> 12)) sc_rc<MODE, E64>(s, P, qs.w, rr, pat);
        rm = 0u;
        continue;
      }
      const uint32_t j = __ffs(em | rm) - 1u;
      if ((em >> j) & 1u) {
        ev = true;
        break;
      }
      // recompute flags of quad j/4 from op j up to the quad's next event
      const uint32_t qb = j & ~3u;
      const uint32_t nxt = em & (0xfu << qb);
      const uint32_t lim = nxt ? __ffs(nxt) - 1u : qb + 4u;
      const uint32_t seg = rm & ((1u << lim) - 1u);
      sc_rc<MODE, E64>(s, P, lds32(qo + 4u * (4u * ch + (j >> 2))), s.rr(), seg >> qb);
      rm &= ~seg;
    }
    if (!__any_sync(0xffffffffu, ev)) break;
    if (ev) {
      const uint32_t j = __ffs(em) - 1u;
      sc_event<MODE, E64>(s, P, 16u * ch + j, lds8(ent + j), cand, active);
      em &= em - 1u;
    }
  }
  cnt = 0;
  __syncwarp();
}

template <uint32_t MODE, bool E64, int MINB>
__global__ void __launch_bounds__(kThreads, MINB) scan_kernel(const __grid_constant__ EvalParams P) {
  extern __shared__ __align__(128) unsigned char sm_raw[];
  __shared__ __align__(8) uint64_t s_bar[kScSlots][kWarps];
  __shared__ uint64_t s_ck[kWarps];
  __shared__ int64_t s_idx[kWarps];

  const uint32_t lane = threadIdx.x & 31u, warp = threadIdx.x >> 5;
  const uint32_t sb = smem_addr(sm_raw);
  const uint32_t ring = sb + warp * kScWarpBytes;
  const uint32_t wl = ring + kScRingW;                 // warp list base: codes [k][lane]
  const uint32_t lst = wl + lane * 16u;                 // this lane's list entries
  const uint32_t m0l = wl + kScListW + lane * 4u;       // and their chunk << 8 | previous op words
  const uint32_t qo = sb + (uint32_t)kWarps * kScWarpBytes;

  // per-quad recompute signature offsets -> shared memory
  for (uint32_t i = threadIdx.x; i < P.qo_words; i += blockDim.x) sts32(qo + 4u * i, __ldg(P.sqo + i));
  if (lane == 0) {
    for (uint32_t k = 0; k < kScSlots; ++k) mbar_init(smem_addr(&s_bar[k][warp]), 1);
    fence_barrier_init();
  }
  __syncthreads();

  // this warp's tiles: one contiguous range [t0, t1) (balanced split, quotient / remainder from
  // the host)
  const uint32_t gw = blockIdx.x * kWarps + warp;
  const uint32_t t0 = gw * P.tw_q + min(gw, P.tw_r);
  const uint32_t t1 = t0 + P.tw_q + (gw < P.tw_r ? 1u : 0u);
  const uint32_t nch = (uint32_t)P.nch;
  const uint32_t nvl = (uint32_t)P.L - 16u * (nch - 1u);  // valid ops of the last chunk
  const unsigned char *codes = reinterpret_cast<const unsigned char *>(P.codes);
  const uint64_t end = (uint64_t)t1 * nch * 512u;
  uint64_t po = (uint64_t)t0 * nch * 512u;  // producer (lane 0): next byte to copy
  auto issue = [&](uint32_t slot) {
    if (po < end) {
      const uint32_t bytes = (uint32_t)min((uint64_t)kScSlotChunks * 512u, end - po);
      const uint32_t bar = smem_addr(&s_bar[slot][warp]);
      mbar_expect_tx(bar, bytes);
      bulk_g2s(ring + slot * (kScSlotChunks * 512u), codes + po, bytes, bar);
      po += bytes;
    }
  };
  if (lane == 0)
    for (uint32_t k = 0; k < kScSlots; ++k) issue(k);
  __syncwarp();

  uint64_t best_ck = ~0ull;
  int64_t best_idx = INT64_MAX;
  ScCand<E64> s;
  uint32_t t = t0, c = 0, cnt = 0, R = 0;
  int64_t cand = (int64_t)t * 32 + lane;
  bool active = t < t1 && cand < P.n;
  sc_init(s, P, active ? __ldg(P.hdr + cand) : 0ull);
  // a chunk is clean when its 16 codes equal the open run's tp/dp code replicated (R: no
  // head, no recompute flag); a dirty chunk is appended to the lane's list
  auto scan_chunk = [&](const uint4 &w, uint32_t cc, bool force) {
    const uint32_t x = (w.x ^ R) | (w.y ^ R) | (w.z ^ R) | (w.w ^ R);
    if ((x != 0u || force) && active) {
      sts128(lst + 512u * cnt, w);
      // recompute-only: the chunk differs from the open run's code in recompute flags only
      const uint32_t rco = ((x & 0xefefefefu) == 0u && !force) ? kScRcOnly : 0u;
      sts32(m0l + 128u * cnt, (cc << 8) | (R & 0xffu) | rco);
      ++cnt;
      R = __byte_perm(w.w, 0u, 0x3333u) & 0xeeeeeeeeu;
    }
  };
  const uint32_t nq = (t1 - t0) * nch;  // chunks of this warp
  uint32_t slot = 0, phase = 0, k = 0;
  uint32_t sa = ring + lane * 16u;  // this lane's 16 bytes of the current chunk in the ring
#pragma unroll 1
  for (uint32_t q = 0; q < nq; ++q) {
    if (k == 0u) mbar_wait(smem_addr(&s_bar[slot][warp]), phase);
    uint4 w = lds128(sa);
    if (c == nch - 1u && nvl < 16u) w = pad_tail(w, nvl);
    scan_chunk(w, c, c == 0u);
    if (++c == nch) {
      // ---- tile end: drain, close the last run and stage (no p2p_fwd), finish ----
      sc_drain<MODE, E64>(s, P, cnt, wl, lane, qo, cand, active);
      sc_close_run<MODE, E64>(s, P, (uint32_t)P.L);
      sc_commit<MODE, E64>(s, P, cand, active);
      sc_finish<MODE, E64>(s, P, cand, active, best_ck, best_idx);
      ++t;
      c = 0;
      cand = (int64_t)t * 32 + lane;
      active = t < t1 && cand < P.n;
      sc_init(s, P, active ? __ldg(P.hdr + cand) : 0ull);
    } else if ((c & 1u) == 0u) {
      if (__any_sync(0xffffffffu, cnt + 2u > kScCap)) sc_drain<MODE, E64>(s, P, cnt, wl, lane, qo, cand, active);
    }
    sa += 512u;
    if (++k == kScSlotChunks || q + 1u == nq) {
      // slot consumed: refill it with the next bytes of this warp's range
      __syncwarp();
      if (lane == 0) {
        fence_proxy_async();
        issue(slot);
      }
      k = 0;
      slot ^= 1u;
      phase ^= slot ^ 1u;  // flips after slot 1
      sa = ring + slot * (kScSlotChunks * 512u) + lane * 16u;
    }
  }

  if (MODE & kSelect) warp_select_finish(best_ck, best_idx, P.sel, P.n_total, P.ib, s_ck, s_idx, P.gkey);
}

}  // namespace aceso
