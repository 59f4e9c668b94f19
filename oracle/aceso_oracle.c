/*
 * aceso_oracle.c — CPU ORACLE (test infrastructure, NOT the product path).
 *
 * A plain, slow, obviously-correct implementation of Aceso's performance and
 * memory model (Liu et al., EuroSys '24, §3.3) and of the selection rule used
 * by its search (Heuristic-1, Alg. 1/2). Only tests/, __graft_entry__.smoke()
 * and bench.py's cpu_baseline / --impl reference legs may load this library.
 * It shares no code, header, table or constant with the CUDA library
 * (paper_conf_eurosys_liumlsmybw24_b200/csrc): the field order, bit layout and
 * reason codes below are restated here from DESIGN.md, not included.
 *
 * "P:Lnn" = line nn of PAPER.md. "R#" = reading #, DESIGN.md §3.
 *
 * Every quantity is an unsigned 64-bit integer (ns or bytes); the model is a
 * definition, so the oracle is that definition written out step by step:
 *   per op   : lookup of the profiled record, recompute adds the forward
 *              to the backward (R7), keeps `keep` bytes (R3)
 *   per stage: S_i, D_i, Wst_i, A_i, E_i (R4, R5, R6, R13)
 *   Eq. 2    : T_i = sum_k S_k + (N-1) S_i + D_i     (R1)
 *   Eq. 1    : Mem_i = Wst_i + min(p-i, N) A_i + E_i (R2, R3, R4)
 *   Heuristic-1: any OOM ? argmax Mem : argmax T, lowest index on ties (R11)
 *   selection: lexicographic min of (class, cost, global index) (R12)
 *
 * Pins (tests/test_oracle_pins.py): 1F1B discrete-event simulation of uniform
 * pipelines (makespan and in-flight activations), closed forms for p = 1 and
 * recomputation, zero-cost-op invariance, Fig. 3 scenarios, record-lookup
 * fingerprints, brute-force enumeration of the toy spaces, and the inter-stage
 * sends (R5) against the 1F1B simulation with sender-side sends on pipelines
 * made uniform by compensating compute, and the DP sync of every stage (R6)
 * against the simulation with a zero-time backward (instant cascade), and the
 * in-stage reshard (R13) against the simulation with the all-gather between the
 * two halves of each microbatch on compensated uniform pipelines.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <pthread.h>

/* --- restated from DESIGN.md §2 (encoding) ------------------------------ */
/* op byte: bit0 head, bits1-3 log2 tp, bit4 recompute, bits5-7 log2 dp      */
/* header : byte0 log2 mbs, byte1 p, bytes2-7 reserved (zero)                */
/* record fields, in order                                                   */
enum { FWD_COMP, FWD_COMM, BWD_COMP, BWD_COMM, ACT, KEEP, PEAK, RESHARD, P2P_FWD, P2P_BWD, NF };
/* info word: bits0-7 bottleneck, 8-15 p, 16 OOM, 17 INVALID, 18.. reasons  */
#define O_OOM (1u << 16)
#define O_INVALID (1u << 17)
/* reasons */
#define O_R_HEAD0 (1u << 0)
#define O_R_NSTAGE (1u << 1)
#define O_R_PRANGE (1u << 2)
#define O_R_GSTAGE (1u << 3)
#define O_R_GSUM (1u << 4)
#define O_R_DPMBS (1u << 5)
#define O_R_TABLE (1u << 6)
#define O_R_MBS (1u << 7)
#define O_R_HDR (1u << 8)

typedef uint64_t u64;

typedef struct {
  int32_t L, T, n_tp, n_dp, n_b, G;
  const uint16_t *op_type;
  const int64_t *rec;  /* [T][n_tp][n_b][NF] */
  const int64_t *rec_alt; /* [T][n_tp][n_b][NF] records of the alternative partition dimension, or 0 */
  const int64_t *wmem; /* [T][n_tp][2] */
  const int64_t *dps;  /* [T][n_tp][n_dp] */
  int64_t C, Bg;
  int literal; /* R1 variant: the literal reading of Eq. 2 */
} oracle_profile;

/* record field of an op of `type` at (tpl, b); dim = 1 reads the records profiled for the
 * op's alternative tensor-parallel partition dimension (§4.2: row- vs
 * column-wise MatMul, input- vs output-channel convolution) */
static u64 rec_field(const oracle_profile *P, int dim, int type, int tpl, int b, int f) {
  const int64_t *r = dim ? P->rec_alt : P->rec;
  return (u64)r[(((int64_t)type * P->n_tp + tpl) * P->n_b + b) * NF + f];
}

/* Evaluates one candidate. codes: [L] bytes, hdr: header. Stage outputs (if
 * non-null) are rows of p_max entries for this candidate. */
static void eval_one(const oracle_profile *P, const uint8_t *codes, const uint8_t *dims, u64 hdr, int32_t p_max,
                     u64 *iter_out, u64 *mem_out, uint32_t *info_out, u64 *sT, u64 *sM, u64 *sC,
                     u64 *sK) {
  const int L = P->L;
  unsigned mbs_log2 = (unsigned)(hdr & 0xff);
  unsigned p = (unsigned)((hdr >> 8) & 0xff);
  uint32_t reasons = 0;

  /* --- header checks ---------------------------------------------------- */
  if (hdr >> 16) reasons |= O_R_HDR;
  u64 N = 0;
  if (mbs_log2 >= 62 || ((u64)1 << mbs_log2) > (u64)P->Bg || ((u64)P->Bg % ((u64)1 << mbs_log2)) != 0)
    reasons |= O_R_MBS;
  else
    N = (u64)P->Bg >> mbs_log2; /* number of microbatches, R8 */
  if (p == 0 || p > (unsigned)P->G) reasons |= O_R_PRANGE;

  /* --- decode every op -------------------------------------- */
  int *head = (int *)malloc(sizeof(int) * L);
  int *tpl = (int *)malloc(sizeof(int) * L);
  int *dpl = (int *)malloc(sizeof(int) * L);
  int *rc = (int *)malloc(sizeof(int) * L);
  int *dim = (int *)malloc(sizeof(int) * L);
  for (int j = 0; j < L; ++j) {
    uint8_t c = codes[j];
    head[j] = c & 1;
    tpl[j] = (c >> 1) & 7;
    rc[j] = (c >> 4) & 1;
    dpl[j] = (c >> 5) & 7;
    dim[j] = dims ? (dims[j] != 0) : 0; /* tensor-parallel partition dimension of op j */
  }

  /* --- structural checks ------------------------------------------------- */
  if (!head[0]) reasons |= O_R_HEAD0;
  unsigned nheads = 0;
  for (int j = 0; j < L; ++j) nheads += (unsigned)head[j];
  if (nheads != p) reasons |= O_R_NSTAGE;
  for (int j = 0; j < L; ++j) {
    if (dpl[j] > (int)mbs_log2) reasons |= O_R_DPMBS;
    if (tpl[j] >= P->n_tp || dpl[j] >= P->n_dp) reasons |= O_R_TABLE;
    if (dpl[j] <= (int)mbs_log2 && (int)mbs_log2 - dpl[j] >= P->n_b) reasons |= O_R_TABLE;
  }
  /* in-stage symmetry: tp*dp constant inside a stage; a stage is op 0's
     segment or starts at an op with head = 1 */
  for (int j = 1; j < L; ++j)
    if (!head[j] && tpl[j] + dpl[j] != tpl[j - 1] + dpl[j - 1]) reasons |= O_R_GSTAGE;
  /* all devices used exactly once (R9) */
  {
    u64 gsum = 0;
    for (int j = 0; j < L; ++j)
      if (j == 0 || head[j]) gsum += (u64)1 << (tpl[j] + dpl[j]);
    if (gsum != (u64)P->G) reasons |= O_R_GSUM;
  }

  if (reasons) {
    *iter_out = 0;
    *mem_out = 0;
    *info_out = (p << 8) | O_INVALID | (reasons << 18);
    free(head); free(tpl); free(dpl); free(rc); free(dim);
    return;
  }

  /* --- per-op costs (valid candidate) ------------------------------------- */
  /* stage id of each op */
  int *sid = (int *)malloc(sizeof(int) * L);
  {
    int s = -1;
    for (int j = 0; j < L; ++j) {
      if (head[j]) s++;
      sid[j] = s;
    }
  }
  u64 *S = (u64 *)calloc(p, sizeof(u64));    /* per-microbatch stage time incl. p2p */
  u64 *Dd = (u64 *)calloc(p, sizeof(u64));   /* DP gradient sync, once per iteration */
  u64 *Wst = (u64 *)calloc(p, sizeof(u64));  /* parameters + grads + optimizer */
  u64 *A = (u64 *)calloc(p, sizeof(u64));    /* activation bytes per in-flight microbatch */
  u64 *E = (u64 *)calloc(p, sizeof(u64));    /* allocator extra = max op transient */
  u64 *comp = (u64 *)calloc(p, sizeof(u64)); /* per-microbatch compute part of S */
  u64 *comm = (u64 *)calloc(p, sizeof(u64)); /* per-microbatch communication part of S */

  for (int j = 0; j < L; ++j) {
    int i = sid[j];
    int t = P->op_type[j];
    int b = (int)mbs_log2 - dpl[j]; /* per-GPU batch = mbs / dp (R8) */
    u64 fc = rec_field(P, dim[j], t, tpl[j], b, FWD_COMP);
    u64 fm = rec_field(P, dim[j], t, tpl[j], b, FWD_COMM);
    u64 bc = rec_field(P, dim[j], t, tpl[j], b, BWD_COMP);
    u64 bm = rec_field(P, dim[j], t, tpl[j], b, BWD_COMM);
    u64 act = rec_field(P, dim[j], t, tpl[j], b, ACT);
    u64 keep = rec_field(P, dim[j], t, tpl[j], b, KEEP);
    u64 peak = rec_field(P, dim[j], t, tpl[j], b, PEAK);
    u64 F = fc + fm;                           /* forward of one microbatch */
    u64 Bp = bc + bm + (rc[j] ? F : 0);        /* recompute adds the forward (R7) */
    u64 Aj = rc[j] ? keep : act;               /* R3 */
    u64 ej = peak + (rc[j] ? (act - keep) : 0); /* R3 + R4 */
    u64 Wj = (u64)P->wmem[((int64_t)t * P->n_tp + tpl[j]) * 2 + 0] +
             (u64)P->wmem[((int64_t)t * P->n_tp + tpl[j]) * 2 + 1];
    u64 dj = (u64)P->dps[((int64_t)t * P->n_tp + tpl[j]) * P->n_dp + dpl[j]];
    u64 rs = 0; /* P:L261, R13: reshard when the tp/dp mix changes inside a stage */
    if (j > 0 && !head[j] && (tpl[j] != tpl[j - 1] || dpl[j] != dpl[j - 1]))
      rs = rec_field(P, dim[j], t, tpl[j], b, RESHARD);
    S[i] += F + Bp + rs;
    comp[i] += fc + bc + (rc[j] ? fc : 0);
    comm[i] += fm + bm + (rc[j] ? fm : 0) + rs;
    Dd[i] += dj;
    Wst[i] += Wj;
    A[i] += Aj;
    if (ej > E[i]) E[i] = ej;
  }
  /* p2p between consecutive stages, paid by the sender (R5) */
  for (unsigned i = 0; i < p; ++i) {
    int first = -1, last = -1;
    for (int j = 0; j < L; ++j)
      if (sid[j] == (int)i) {
        if (first < 0) first = j;
        last = j;
      }
    if (i + 1 < p) {
      int t = P->op_type[last];
      u64 v = rec_field(P, dim[last], t, tpl[last], (int)mbs_log2 - dpl[last], P2P_FWD);
      S[i] += v;
      comm[i] += v;
    }
    if (i > 0) {
      int t = P->op_type[first];
      u64 v = rec_field(P, dim[first], t, tpl[first], (int)mbs_log2 - dpl[first], P2P_BWD);
      S[i] += v;
      comm[i] += v;
    }
  }

  /* --- Eq. 2 (R1) and Eq. 1 (R2) ----------------------------------------- */
  u64 sumS = 0;
  for (unsigned i = 0; i < p; ++i) sumS += S[i];
  u64 iter = 0, maxmem = 0;
  unsigned argT = 0, argM = 0;
  int oom = 0;
  for (unsigned i = 0; i < p; ++i) {
    u64 Ti = sumS + (N - 1) * S[i] + Dd[i];
    if (P->literal) Ti += S[i]; /* R1 variant: Eq. 2 as printed (steady phase N, not N-1, microbatches) */
    u64 inflight = (u64)(p - i) < N ? (u64)(p - i) : N;
    u64 Mi = Wst[i] + inflight * A[i] + E[i];
    if (Mi > (u64)P->C) oom = 1; /* R10 */
    if (i == 0 || Ti > iter) { iter = Ti; argT = i; }
    if (i == 0 || Mi > maxmem) { maxmem = Mi; argM = i; }
    if (sT) sT[i] = Ti;
    if (sM) sM[i] = Mi;
    if (sC) sC[i] = N * comp[i];
    if (sK) sK[i] = N * comm[i] + Dd[i];
  }
  (void)p_max;
  unsigned bottleneck = oom ? argM : argT; /* Heuristic-1 */
  *iter_out = iter;
  *mem_out = maxmem;
  *info_out = bottleneck | (p << 8) | (oom ? O_OOM : 0);

  free(sid); free(S); free(Dd); free(Wst); free(A); free(E); free(comp); free(comm);
  free(head); free(tpl); free(dpl); free(rc); free(dim);
}

typedef struct {
  const oracle_profile *P;
  const uint8_t *codes;
  const uint8_t *dims;
  const uint64_t *hdr;
  int64_t lo, hi;
  int32_t p_max;
  uint64_t *iter, *mem, *sT, *sM, *sC, *sK;
  uint32_t *info;
} job_t;

static void *run_job(void *arg) {
  job_t *J = (job_t *)arg;
  for (int64_t c = J->lo; c < J->hi; ++c) {
    int64_t o = c * J->p_max;
    eval_one(J->P, J->codes + c * (int64_t)J->P->L, J->dims ? J->dims + c * (int64_t)J->P->L : 0,
             J->hdr[c], J->p_max, &J->iter[c], &J->mem[c],
             &J->info[c], J->sT ? J->sT + o : 0, J->sM ? J->sM + o : 0, J->sC ? J->sC + o : 0,
             J->sK ? J->sK + o : 0);
  }
  return 0;
}

/* Public entry: evaluates n candidates (row-major codes [n][L]) on n_threads
 * host threads (contiguous blocks). rec_alt / dims (nullable): records of each op type's
 * alternative tensor-parallel partition dimension and the per-op choice (row-major [n][L],
 * nonzero = alternative; dims require rec_alt). Stage arrays are [n][p_max] (nullable);
 * entries i >= p are left untouched; for invalid candidates nothing is written.
 * Returns 0, or -1 on bad arguments. */
int oracle_eval(int32_t L, int32_t T, int32_t n_tp, int32_t n_dp, int32_t n_b, int32_t G,
                const uint16_t *op_type, const int64_t *rec, const int64_t *rec_alt, const int64_t *wmem,
                const int64_t *dps, int64_t C, int64_t Bg, const uint8_t *codes, const uint8_t *dims,
                const uint64_t *hdr, int64_t n, int32_t p_max, uint64_t *iter, uint64_t *max_mem,
                uint32_t *info, uint64_t *stage_T, uint64_t *stage_mem, uint64_t *stage_comp,
                uint64_t *stage_comm, int n_threads, int literal) {
  if (L < 1 || T < 1 || n < 0 || !op_type || !rec || !wmem || !dps || (n && (!codes || !hdr)))
    return -1;
  if ((stage_T || stage_mem || stage_comp || stage_comm) && p_max < G) return -1;
  if (dims && !rec_alt) return -1;
  oracle_profile P = {L, T, n_tp, n_dp, n_b, G, op_type, rec, rec_alt, wmem, dps, C, Bg, literal};
  if (n_threads < 1) n_threads = 1;
  if (n_threads > 256) n_threads = 256;
  if ((int64_t)n_threads > n) n_threads = n > 0 ? (int)n : 1;
  job_t jobs[256];
  pthread_t th[256];
  for (int k = 0; k < n_threads; ++k) {
    jobs[k] = (job_t){&P, codes, dims, hdr, n * k / n_threads, n * (k + 1) / n_threads, p_max,
                      iter, max_mem, stage_T, stage_mem, stage_comp, stage_comm, info};
  }
  if (n_threads == 1) {
    run_job(&jobs[0]);
    return 0;
  }
  for (int k = 0; k < n_threads; ++k) pthread_create(&th[k], 0, run_job, &jobs[k]);
  for (int k = 0; k < n_threads; ++k) pthread_join(th[k], 0);
  return 0;
}

/* Selection over evaluated candidates ("better"; Alg. 1 GetBestOf):
 * class 0 (feasible, cost = iteration time) before class 1 (OOM, cost = max
 * memory, R12), then lower cost, then lower global index (R11). Invalid
 * candidates are skipped. Writes *index = -1 when nothing is valid. */
void oracle_select(const uint64_t *iter, const uint64_t *max_mem, const uint32_t *info, int64_t n,
                   int64_t global_offset, int *cls, uint64_t *cost, int64_t *index) {
  int best_cls = -1;
  u64 best_cost = 0;
  int64_t best_idx = -1;
  for (int64_t c = 0; c < n; ++c) {
    if (info[c] & O_INVALID) continue;
    int k = (info[c] & O_OOM) ? 1 : 0;
    u64 v = k ? max_mem[c] : iter[c];
    int64_t g = global_offset + c;
    int better = 0;
    if (best_idx < 0) better = 1;
    else if (k != best_cls) better = k < best_cls;
    else if (v != best_cost) better = v < best_cost;
    else better = g < best_idx;
    if (better) { best_cls = k; best_cost = v; best_idx = g; }
  }
  *cls = best_cls;
  *cost = best_cost;
  *index = best_idx;
}
