// incr_kernel.cuh — incremental evaluation of candidates given as base + patches (SURVEY
// §8(f) NEXT(2): "re-reduce only the touched stages").
//
// A reconfiguration primitive rewrites a few byte ranges of its base configuration
// (include/aceso.h, aceso_cand). A stage's sums depend only on its own ops and boundaries,
// so every stage that no patch range [a-1, b) overlaps keeps the base's per-stage values.
// base_cache_kernel walks each base once and stores, per stage: S_i, D_i, comp_i, the Eq. 2
// key (N-1) S_i + D_i, Mem_i (Eq. 1), its device group g_i and its first op, plus an op ->
// stage map. incr_kernel folds the stages of a candidate in index order: cached values for
// untouched stages, a per-op walk (the model's definition: record lookup by (type, tp,
// per-GPU batch), recompute, reshard, p2p) over each run of touched stages. A candidate whose
// microbatch or stage count differs from its base, or whose base is invalid or has more than
// 64 stages, is walked over all ops (same code, every stage touched).
//
// The candidate walk (walk_events) is event-driven like event_kernel.cuh: it patches the
// base's codes 16 ops at a time, finds the chunk's events (stage heads, tp/dp changes) and
// recompute flags with the activity words, and takes every run's sums from the position-
// prefix tables (PX, PD, sparse-table range max ST, recompute deltas QR per quad pattern),
// so a touched stage costs O(its chunks + its events), not a table walk per op.
//
// Paper: Eq. 1, Eq. 2, Heuristic-1, readings R1-R13, R18-R20.
#pragma once
#include "common.cuh"
#include "eval_kernel.cuh"    // kSummary / kFull / kSelect
#include "event_kernel.cuh"   // activity words, event / recompute masks, event tables
#include "expand_kernel.cuh"  // patched_chunk

namespace aceso {

struct IncrBaseHdr {   // 32 bytes
  uint32_t p, reasons, mbs, N;
  uint64_t sumS, pad;
};
struct IncrBaseStage {  // 48 bytes
  uint64_t S, D, comp, keyT, mem;
  uint32_t g, head;
};

// one stage being accumulated by the walk
struct WalkStage {
  uint64_t S, A, W, D, comp;
  uint32_t E, g, head;
};

// Event-driven walk of ops [A, B) of a candidate (A is a segment start: a stage starts at A
// whatever its head bit, R19; B = L or a head): same stages, same emit order and same
// per-op validity as a walk over every op would give, from the event tables. Sums are kept in prefix-difference
// form (exact mod 2^64). Returns the number of head bits walked.
template <bool FULL, class Emit>
__device__ __forceinline__ uint32_t walk_events(const EvalParams &P, const uint4 *__restrict__ brow,
                                                const uint16_t *__restrict__ ranks, uint32_t base,
                                                const aceso_cand &cd, int np, uint32_t mbs, uint32_t A,
                                                uint32_t B, Emit emit, uint32_t *reasons) {
  const uint32_t L = (uint32_t)P.L, Lp1 = L + 1u, NT = (uint32_t)P.n_tp, NB = (uint32_t)P.n_b;
  const int32_t stride = 16 * (int32_t)((L + 15u) / 16u);
  const uint32_t *qo = reinterpret_cast<const uint32_t *>(P.evblob + P.qo_off);
  WalkStage st;
  st.S = st.A = st.W = st.D = st.comp = 0;
  st.E = 0;
  st.g = 0;
  st.head = A;
  uint32_t rr = 0, dd = 0, ra = A, nst = 0;
  // closes the open run [ra, j) (prefix differences, range max R4)
  auto close_run = [&](uint32_t j) {
    const uint32_t o = rr * Lp1 + j;
    const uint4 x0 = __ldg(P.px + 2u * o);
    const uint4 x1 = __ldg(P.px + 2u * o + 1u);
    const uint32_t k = 31u - __clz(j - ra);
    const uint32_t *stk = P.st + ((k * (uint32_t)P.runs + rr) * L);
    st.S += u64of(x0.x, x0.y);
    st.A += u64of(x0.z, x0.w);
    st.W += u64of(x1.x, x1.y);
    if (FULL) st.comp += u64of(x1.z, x1.w);
    st.D += __ldg(P.pd + (dd * Lp1 + j));
    st.E = max(st.E, max(__ldg(stk + ra), __ldg(stk + (j - (1u << k)))));
  };
  const uint32_t *kx = reinterpret_cast<const uint32_t *>(P.kx);
  uint32_t pw = 0;
  const uint32_t c0 = A >> 4, c1 = (B - 1u) >> 4;
  if (c0 > 0) pw = patched_chunk(brow, ranks, base, stride, (int32_t)L, cd, np, (int32_t)c0 - 1).w;
  for (uint32_t ch = c0; ch <= c1; ++ch) {
    const uint4 w4 = patched_chunk(brow, ranks, base, stride, (int32_t)L, cd, np, (int32_t)ch);
    uint4 f;
    f.x = quad_activity(w4.x, pw);
    f.y = quad_activity(w4.y, w4.x);
    f.z = quad_activity(w4.z, w4.y);
    f.w = quad_activity(w4.w, w4.z);
    pw = w4.w;
    const bool edge = ch == c0 || ch == c1;
    if (!edge && (f.x | f.y | f.z | f.w) == 0u) continue;  // no event, no recompute flag
    uint32_t em = ev_event_mask(f), rm = ev_rc_mask(f);
    if (edge) {
      // ops of the chunk inside [A, B); op A is always an event (segment start)
      const uint32_t lo = ch == c0 ? (A & 15u) : 0u, hi = ch == c1 ? ((B - 1u) & 15u) + 1u : 16u;
      const uint32_t in = (hi >= 16u ? 0xffffu : ((1u << hi) - 1u)) & ~((1u << lo) - 1u);
      em = (em | (ch == c0 ? (1u << lo) : 0u)) & in;
      rm &= in;
    }
    while (em | rm) {
      const uint32_t j = __ffs(em | rm) - 1u;
      const uint32_t op = 16u * ch + j;
      if ((em >> j) & 1u) {
        const uint32_t wq = (j >> 2) == 0u ? w4.x : (j >> 2) == 1u ? w4.y : (j >> 2) == 2u ? w4.z : w4.w;
        const uint32_t c = (wq >> (8u * (j & 3u))) & 0xffu;
        const uint32_t head = c & 1u, tpl = (c >> 1) & 7u, dpl = c >> 5;
        if (dpl > mbs) *reasons |= ACESO_R_DPMBS;
        if (tpl >= NT || dpl >= (uint32_t)P.n_dp || (dpl <= mbs && mbs - dpl >= NB)) *reasons |= ACESO_R_TABLE;
        // clamped indices keep every gather inside the tables for invalid encodings
        const uint32_t b = min(dpl <= mbs ? mbs - dpl : 0u, NB - 1);
        const uint32_t tplc = min(tpl, NT - 1), dplc = min(dpl, (uint32_t)P.n_dp - 1);
        const uint32_t rn = b * NT + tplc;
        const uint32_t on = rn * Lp1 + op;
        if (op == A || head) {
          if (op > A) {  // close the stage: its last run, p2p_fwd of its last op (R5)
            close_run(op);
            st.S += __ldg(kx + (4u * (rr * Lp1 + op) + 2u));
            emit(st);
          }
          st.S = st.A = st.W = st.D = st.comp = 0;
          st.E = 0;
          st.g = tpl + dpl;
          st.head = op;
          nst += head;
          if (op > 0 && head) st.S += __ldg(kx + (4u * on + 1u));  // p2p_bwd of the first op (R5)
        } else {
          close_run(op);
          if (tpl + dpl != st.g) *reasons |= ACESO_R_GSTAGE;
          st.S += __ldg(kx + 4u * on);                        // reshard into this op (R13)
        }
        // open the run of op `op`
        const uint4 y0 = __ldg(P.px + 2u * on);
        const uint4 y1 = __ldg(P.px + 2u * on + 1u);
        st.S -= u64of(y0.x, y0.y);
        st.A -= u64of(y0.z, y0.w);
        st.W -= u64of(y1.x, y1.y);
        if (FULL) st.comp -= u64of(y1.z, y1.w);
        rr = rn;
        dd = tplc * (uint32_t)P.n_dp + dplc;
        st.D -= __ldg(P.pd + (dd * Lp1 + op));
        ra = op;
        em &= em - 1u;
      } else {
        // recompute flags of quad j/4 from op j up to the quad's next event, under the open
        // run (R3, R4, R7)
        const uint32_t qb = j & ~3u;
        const uint32_t nxt = em & (0xfu << qb);
        const uint32_t lim = nxt ? __ffs(nxt) - 1u : qb + 4u;
        const uint32_t seg = rm & ((1u << lim) - 1u);
        uint64_t dS = 0, dA = 0, dC = 0;
        uint32_t e1 = 0;
        ev_rc_lookup<FULL ? kFull : 0u>(P, __ldg(qo + 4u * ch + (j >> 2)), rr, seg >> qb, dS, dA, e1, dC);
        st.S += dS;
        st.A -= dA;
        st.E = max(st.E, e1);
        if (FULL) st.comp += dC;
        rm &= ~seg;
      }
    }
  }
  close_run(B);
  if (B < L) st.S += __ldg(kx + (4u * (rr * Lp1 + B) + 2u));  // followed by a stage (R5, R20)
  emit(st);
  return nst;
}

__device__ __forceinline__ uint32_t header_reasons(uint64_t h, const EvalParams &P, uint32_t *N) {
  const uint32_t mbs = (uint32_t)(h & 0xff), p = (uint32_t)((h >> 8) & 0xff);
  uint32_t reasons = (h >> 16) ? ACESO_R_HDR : 0u;
  *N = 0;
  if (mbs >= 62 || (1ull << mbs) > P.Bg || (P.Bg & ((1ull << mbs) - 1)) != 0) reasons |= ACESO_R_MBS;
  else *N = (uint32_t)(P.Bg >> mbs);
  if (p == 0 || p > (uint32_t)P.G) reasons |= ACESO_R_PRANGE;
  return reasons;
}

// One thread per base: per-stage cache and op -> stage map (workspace of include/aceso.h).
__global__ void __launch_bounds__(128) base_cache_kernel(const __grid_constant__ EvalParams P,
                                                         const uint8_t *__restrict__ bases,
                                                         const uint64_t *__restrict__ base_hdr,
                                                         int32_t nb, IncrBaseHdr *hdrs,
                                                         IncrBaseStage *stages, uint8_t *smap) {
  const int32_t b = blockIdx.x * blockDim.x + threadIdx.x;
  if (b >= nb) return;
  const uint32_t L = (uint32_t)P.L, stride = 16u * (((uint32_t)P.L + 15u) / 16u);
  const uint8_t *row = bases + (size_t)b * stride;
  const uint64_t hb = base_hdr[b];
  const uint32_t mbs = (uint32_t)(hb & 0xff), p = (uint32_t)((hb >> 8) & 0xff);
  uint32_t N = 0;
  uint32_t reasons = header_reasons(hb, P, &N);
  IncrBaseStage *out = stages + (size_t)b * P.G;
  uint64_t sumS = 0;
  uint32_t i = 0, gsum = 0;
  auto emit = [&](const WalkStage &s) {
    if (i < (uint32_t)P.G) {
      const uint64_t infl = p > i ? (uint64_t)min(p - i, N) : 0ull;
      IncrBaseStage r;
      r.S = s.S;
      r.D = s.D;
      r.comp = s.comp;
      r.keyT = (uint64_t)(N - 1) * s.S + s.D;
      r.mem = (s.W + infl * s.A + s.E) << P.mem_shift;
      r.g = s.g;
      r.head = s.head;
      out[i] = r;
    }
    for (uint32_t j = s.head; j < L && (j == s.head || !(row[j] & 1u)); ++j) smap[(size_t)b * L + j] = (uint8_t)min(i, 255u);
    sumS += s.S;
    gsum += 1u << s.g;
    i += 1;
  };
  aceso_cand cd0;
  memset(&cd0, 0, sizeof(cd0));  // no patches: the base itself
  const uint32_t nst = walk_events<true>(P, reinterpret_cast<const uint4 *>(row), nullptr, (uint32_t)b, cd0, 0, mbs,
                                         0, L, emit, &reasons);
  if (!(row[0] & 1u)) reasons |= ACESO_R_HEAD0;
  if (nst != p) reasons |= ACESO_R_NSTAGE;
  if (gsum != (uint32_t)P.G) reasons |= ACESO_R_GSUM;
  IncrBaseHdr h;
  h.p = p;
  h.reasons = reasons;
  h.mbs = mbs;
  h.N = N;
  h.sumS = sumS;
  h.pad = 0;
  hdrs[b] = h;
}

// One thread per candidate: fold cached and re-walked stages in index order.
template <uint32_t MODE>
__global__ void __launch_bounds__(256) incr_kernel(const __grid_constant__ EvalParams P,
                                                   const uint8_t *__restrict__ bases,
                                                   const uint16_t *__restrict__ ranks, int32_t nb,
                                                   const aceso_cand *__restrict__ cands,
                                                   const IncrBaseHdr *__restrict__ hdrs,
                                                   const IncrBaseStage *__restrict__ stages,
                                                   const uint8_t *__restrict__ smap) {
  __shared__ uint64_t s_ck[kWarps];
  __shared__ int64_t s_idx[kWarps];
  const uint32_t L = (uint32_t)P.L, stride = 16u * ((L + 15u) / 16u);
  uint64_t best_ck = ~0ull;
  int64_t best_idx = INT64_MAX;
  for (int64_t c = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; c - (threadIdx.x & 31) < P.n;
       c += (int64_t)gridDim.x * blockDim.x) {
    if (c >= P.n) continue;
    const aceso_cand cd = cands[c];
    const uint32_t base = min(cd.base, (uint32_t)nb - 1u);
    const uint8_t *row = bases + (size_t)base * stride;
    const uint32_t mbs = cd.mbs_log2, p = cd.p;
    uint32_t N = 0;
    uint32_t reasons = header_reasons((uint64_t)mbs | ((uint64_t)p << 8), P, &N);
    const int np = min((int)cd.n_patch, 6);
    const uint4 *brow = reinterpret_cast<const uint4 *>(row);
    const int32_t stride_i = (int32_t)stride;
    const IncrBaseHdr bh = hdrs[base];
    const bool full = bh.reasons != 0u || bh.mbs != mbs || bh.p != p || p > 64u;
    uint64_t touched = ~0ull;  // stages to re-walk (bit i)
    if (!full) {
      touched = 0;
      for (int k = 0; k < np; ++k) {
        const uint32_t a = min((uint32_t)cd.patch[k].a, L), e = min((uint32_t)cd.patch[k].b, L);
        if (e <= a) continue;
        const uint32_t s1 = __ldg(smap + (size_t)base * L + (a > 0 ? a - 1u : 0u));
        const uint32_t s2 = __ldg(smap + (size_t)base * L + e - 1u);
        touched |= ((s2 >= 63u ? ~0ull : ((2ull << s2) - 1ull))) & ~((1ull << s1) - 1ull);
      }
    }
    // fold stages in index order
    uint64_t sumS = 0, bestT = 0, bestM = 0;
    uint32_t bt = 0, bm = 0, oom = 0, gsum = 0, i = 0, nst = 0;
    const bool act = true;
    auto fold = [&](uint64_t S, uint64_t D, uint64_t comp, uint64_t keyT, uint64_t mem, uint32_t g) {
      sumS += S;
      if (i == 0 || keyT > bestT) { bestT = keyT; bt = i; }  // ties: lowest stage index (R11)
      if (i == 0 || mem > bestM) { bestM = mem; bm = i; }
      oom |= mem > P.C ? 1u : 0u;
      gsum += 1u << g;
      if ((MODE & kFull) && i < (uint32_t)P.p_max) {
        const int64_t o = (int64_t)i * P.n + c;
        P.stage_T[o] = keyT;  // + sum_k S_k below
        P.stage_mem[o] = mem;
        P.stage_comp[o] = (uint64_t)N * comp;
        P.stage_comm[o] = (uint64_t)N * (S - comp) + D;
      }
      i += 1;
    };
    auto emit = [&](const WalkStage &s) {
      const uint64_t infl = p > i ? (uint64_t)min(p - i, N) : 0ull;
      fold(s.S, s.D, s.comp, (uint64_t)(N - 1) * s.S + s.D, (s.W + infl * s.A + s.E) << P.mem_shift, s.g);
    };
    const uint32_t op0 = patched_chunk(brow, ranks, base, stride_i, (int32_t)L, cd, np, 0).x & 0xffu;
    if (full) {
      nst = walk_events<(MODE & kFull) != 0>(P, brow, ranks, base, cd, np, mbs, 0, L, emit, &reasons);
    } else {
      const IncrBaseStage *bs = stages + (size_t)base * P.G;
      uint32_t s = 0;
      while (s < bh.p) {
        if (!((touched >> s) & 1ull)) {
          const IncrBaseStage r = bs[s];
          fold(r.S, r.D, r.comp, r.keyT, r.mem, r.g);
          nst += 1;
          s += 1;
          continue;
        }
        uint32_t e = s;
        while (e + 1 < bh.p && ((touched >> (e + 1)) & 1ull)) e += 1;
        const uint32_t A = bs[s].head, B = e + 1 < bh.p ? bs[e + 1].head : L;
        nst += walk_events<(MODE & kFull) != 0>(P, brow, ranks, base, cd, np, mbs, A, B, emit, &reasons);
        s = e + 1;
      }
    }
    if (!(op0 & 1u)) reasons |= ACESO_R_HEAD0;
    if (nst != p) reasons |= ACESO_R_NSTAGE;
    if (gsum != (uint32_t)P.G) reasons |= ACESO_R_GSUM;
    // epilogue (as finish_cand): validity, summary, FULL, fused argmin
    const bool invalid = reasons != 0u;
    const uint64_t iter = invalid ? 0ull : sumS + bestT;
    const uint64_t mem = invalid ? 0ull : bestM;
    uint32_t info = p << 8;
    if (invalid) info |= ACESO_INFO_INVALID | (reasons << 18);
    else info |= oom ? (bm | ACESO_INFO_OOM) : bt;
    if (MODE & kSummary) {
      P.iter_ns[c] = iter;
      P.max_mem[c] = mem;
      P.info[c] = info;
    }
    if ((MODE & kFull) && !invalid) {
      const uint32_t ns = min(p, (uint32_t)P.p_max);
      for (uint32_t k = 0; k < ns; ++k) P.stage_T[(int64_t)k * P.n + c] += sumS;
    }
    if ((MODE & kSelect) && !invalid && act) {
      const uint64_t ck = oom ? ((1ull << 62) | mem) : iter;
      const int64_t g = P.gofs + c;
      if (key_less(ck, g, best_ck, best_idx)) {
        best_ck = ck;
        best_idx = g;
      }
    }
  }
  if (MODE & kSelect) warp_select_finish(best_ck, best_idx, P.sel, P.n_total, P.ib, s_ck, s_idx);
}

}  // namespace aceso
