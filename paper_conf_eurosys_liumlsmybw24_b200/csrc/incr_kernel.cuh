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
// Paper: Eq. 1, Eq. 2, Heuristic-1, readings R1-R13, R18-R20.
#pragma once
#include "common.cuh"
#include "eval_kernel.cuh"  // kSummary / kFull / kSelect

namespace aceso {

struct IncrBaseHdr {   // 32 bytes
  uint32_t p, reasons, mbs, N;
  uint64_t sumS, pad;
};
struct IncrBaseStage {  // 48 bytes
  uint64_t S, D, comp, keyT, mem;
  uint32_t g, head;
};

struct IncrTabs {
  const uint32_t *R, *D, *F, *K;  // packed per-op tables of the blob (eval_kernel.cuh layout)
  const uint16_t *T;              // op types
  uint32_t nT;
};

__device__ __forceinline__ IncrTabs incr_tabs(const EvalParams &P) {
  const unsigned char *blob = reinterpret_cast<const unsigned char *>(P.blob);
  IncrTabs t;
  t.R = reinterpret_cast<const uint32_t *>(blob + P.tab.offR);
  t.D = reinterpret_cast<const uint32_t *>(blob + P.tab.offD);
  t.F = reinterpret_cast<const uint32_t *>(blob + P.tab.offF);
  t.K = reinterpret_cast<const uint32_t *>(blob + P.tab.offK);
  t.T = reinterpret_cast<const uint16_t *>(blob + P.tab.offT);
  t.nT = (uint32_t)P.T;
  return t;
}

// one stage being accumulated by the walk
struct WalkStage {
  uint64_t S, A, W, D, comp;
  uint32_t E, g, head;
};

// Walks ops [A, B) (A is a stage start, B = L or a head) of the configuration code_at(j),
// calling emit(stage) for every stage it closes, in order. Per-op validity goes to *reasons;
// returns the number of head bits walked.
template <bool FULL, class CodeAt, class Emit>
__device__ __forceinline__ uint32_t walk_ops(const EvalParams &P, const IncrTabs &t, uint32_t mbs,
                                             uint32_t A, uint32_t B, CodeAt code_at, Emit emit,
                                             uint32_t *reasons) {
  const uint32_t NT = (uint32_t)P.n_tp, NB = (uint32_t)P.n_b;
  WalkStage st;
  uint32_t nst = 0, pc = 0, prt = 0;  // previous op's code and (run, type) index
  for (uint32_t j = A; j < B; ++j) {
    const uint32_t c = code_at(j);
    const uint32_t head = c & 1u, tpl = (c >> 1) & 7u, rc = (c >> 4) & 1u, dpl = c >> 5;
    if (dpl > mbs) *reasons |= ACESO_R_DPMBS;
    if (tpl >= NT || dpl >= (uint32_t)P.n_dp || (dpl <= mbs && mbs - dpl >= NB)) *reasons |= ACESO_R_TABLE;
    const uint32_t b = min(dpl <= mbs ? mbs - dpl : 0u, NB - 1);
    const uint32_t tplc = min(tpl, NT - 1);
    const uint32_t type = __ldg(t.T + j);
    const uint32_t rt = (b * NT + tplc) * t.nT + type;  // (run, type) record index
    if (j == A || head) {
      if (j > A) {  // close the previous stage: p2p_fwd of its last op (R5)
        st.S += __ldg(t.K + prt * 4 + 1);
        emit(st);
      }
      st.S = st.A = st.W = st.D = st.comp = 0;
      st.E = 0;
      st.g = tpl + dpl;
      st.head = j;
      nst += head;  // NSTAGE counts head bits (op 0 starts a segment even without one, R19)
      if (j > 0 && head) st.S += __ldg(t.K + rt * 4 + 2);  // p2p_bwd of the stage's first op (R5)
    } else {
      if (tpl + dpl != st.g) *reasons |= ACESO_R_GSTAGE;
      if (((c ^ pc) & 0xEEu) != 0u) st.S += __ldg(t.K + rt * 4);  // reshard into this op (R13)
    }
    const uint4 r = __ldg(reinterpret_cast<const uint4 *>(t.R + rt * 8 + rc * 4));
    st.S += r.x;
    st.A += r.y;
    st.E = max(st.E, r.z);
    st.W += r.w;
    st.D += __ldg(t.D + (tplc * t.nT + type) * 8 + dpl);
    if (FULL) st.comp += __ldg(t.F + rt * 2 + rc);
    pc = c;
    prt = rt;
  }
  if (B < (uint32_t)P.L) st.S += __ldg(t.K + prt * 4 + 1);  // followed by a stage (R5, R20)
  if (B > A) emit(st);
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
  const IncrTabs t = incr_tabs(P);
  const uint32_t L = (uint32_t)P.L, stride = 16u * (((uint32_t)P.L + 15u) / 16u);
  const uint8_t *row = bases + (size_t)b * stride;
  const uint64_t hb = base_hdr[b];
  const uint32_t mbs = (uint32_t)(hb & 0xff), p = (uint32_t)((hb >> 8) & 0xff);
  uint32_t N = 0;
  uint32_t reasons = header_reasons(hb, P, &N);
  IncrBaseStage *out = stages + (size_t)b * P.G;
  uint64_t sumS = 0;
  uint32_t i = 0, gsum = 0;
  auto code_at = [&](uint32_t j) { return (uint32_t)__ldg(row + j); };
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
  const uint32_t nst = walk_ops<true>(P, t, mbs, 0, L, code_at, emit, &reasons);
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
  __shared__ unsigned int s_done;
  if (threadIdx.x == 0) s_done = 0;
  __syncthreads();
  const IncrTabs t = incr_tabs(P);
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
    // the candidate's code at op j: the base's byte with the patches applied in order
    auto code_at = [&](uint32_t j) {
      uint32_t v = __ldg(row + j);
      for (int k = 0; k < np; ++k) {
        const aceso_patch pt = cd.patch[k];
        if (j < pt.a || j >= pt.b) continue;
        if (pt.kind == ACESO_PATCH_MASK) {
          v = (v & pt.v0) | pt.v1;
        } else if (pt.kind == ACESO_PATCH_ADD) {
          v = (v + (uint32_t)(((int)(int8_t)pt.v0 << 1) + ((int)(int8_t)pt.v1 << 5))) & 0xffu;
        } else if (pt.kind == ACESO_PATCH_RANK_RC && ranks != nullptr) {
          const uint32_t kk = (uint32_t)pt.v0 | ((uint32_t)pt.v1 << 8);
          if ((uint32_t)__ldg(ranks + ((size_t)base * 2 + (pt.v2 & 1u)) * stride + j) < kk)
            v = (pt.v2 & 2u) ? (v & 0xefu) : (v | 0x10u);
        }
      }
      return v;
    };
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
    uint32_t op0 = code_at(0);
    if (full) {
      nst = walk_ops<(MODE & kFull) != 0>(P, t, mbs, 0, L, code_at, emit, &reasons);
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
        nst += walk_ops<(MODE & kFull) != 0>(P, t, mbs, A, B, code_at, emit, &reasons);
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
  if (MODE & kSelect) warp_select_finish(best_ck, best_idx, P.sel, P.n_total, P.ib, s_ck, s_idx, &s_done);
}

}  // namespace aceso
