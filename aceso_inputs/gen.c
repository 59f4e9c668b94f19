/*
 * gen.c — seeded synthetic candidate generators (input synthesis only).
 *
 * Shared by the oracle-side tests and the GPU-side tests/bench: it holds none
 * of the method's arithmetic (no cost lookup, no Eq. 1/2, no selection). It
 * only writes configuration encodings:
 *   op byte: bit0 head, bits1-3 log2 tp, bit4 recompute, bits5-7 log2 dp
 *   header : byte0 log2 mbs, byte1 p
 *
 * Randomness is counter-based (splitmix64 of seed and global candidate index),
 * so any shard [first, first+n) of a job regenerates exactly its candidates.
 *
 * Distributions ("input recipe"):
 *  - search-shaped: candidates come in groups sharing a base configuration —
 *    the even partition with minimum microbatch for one stage count
 *    p (parallel search per p) — and each applies 1..7 (MaxHops,
 *    P:L313) random Table-1 primitives: op moves at stage edges
 *    (P:L253), mbs changes, dp/tp trades with a partner stage,
 *    in-stage tp<->dp trades, greedy recomputation of the largest-activation
 *    op types, op-level fine-tuning from op k to the stage end
 *    (P:L261); ~2% are corrupted into invalid encodings.
 *  - dense-random: every op of every stage gets a random (tp, dp) with the
 *    stage's tp*dp, and a random recompute bit (adversarial).
 *  - exhaustive: every configuration of a tiny model, in a fixed order.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

typedef struct {
  int32_t L, n_tp, n_dp, n_b, G;
  int64_t Bg;
  const uint8_t *rc_rank; /* [L] per-op rank of its type by activation size (0 = largest) */
} gen_model;

static inline uint64_t sm64(uint64_t x) {
  x += 0x9E3779B97F4A7C15ull;
  x = (x ^ (x >> 30)) * 0xBF58476D1CE4E5B9ull;
  x = (x ^ (x >> 27)) * 0x94D049BB133111EBull;
  return x ^ (x >> 31);
}
typedef struct { uint64_t s; } rng_t;
static inline rng_t rng_make(uint64_t seed, uint64_t stream, uint64_t idx) {
  rng_t r;
  r.s = sm64(seed ^ sm64(stream * 0xD1B54A32D192ED03ull ^ sm64(idx)));
  return r;
}
static inline uint64_t rng_next(rng_t *r) {
  r->s += 0x9E3779B97F4A7C15ull;
  uint64_t x = r->s;
  x = (x ^ (x >> 30)) * 0xBF58476D1CE4E5B9ull;
  x = (x ^ (x >> 27)) * 0x94D049BB133111EBull;
  return x ^ (x >> 31);
}
static inline uint32_t rng_below(rng_t *r, uint32_t n) { return (uint32_t)(rng_next(r) % n); }

static int ilog2(int64_t v) {
  int k = 0;
  while (((int64_t)1 << (k + 1)) <= v) k++;
  return k;
}

#define MAXP 256

typedef struct {
  int p;
  int mbs_log2;
  int start[MAXP + 1]; /* start[i] = first op of stage i; start[p] = L */
  int tpl[MAXP], dpl[MAXP], rcl[MAXP];
  int ft_from[MAXP]; /* op-level fine-tune: ops >= ft_from get (tpl+ft_d, dpl-ft_d) */
  int ft_d[MAXP];
} cfg_t;

static size_t tiled_off(int64_t c, int j, int nch) {
  return (size_t)(((c / 32) * nch + j / 16) * 512 + (c % 32) * 16 + (j % 16));
}

static void emit(const gen_model *M, const cfg_t *cf, uint8_t *codes, uint64_t *hdr, int64_t c,
                 int tiled) {
  int L = M->L, nch = (L + 15) / 16;
  for (int i = 0; i < cf->p; ++i) {
    for (int j = cf->start[i]; j < cf->start[i + 1]; ++j) {
      int tp = cf->tpl[i], dp = cf->dpl[i];
      if (j >= cf->ft_from[i]) { tp += cf->ft_d[i]; dp -= cf->ft_d[i]; }
      int rc = (int)M->rc_rank[j] < cf->rcl[i] ? 1 : 0;
      uint8_t v = (uint8_t)((j == cf->start[i] ? 1 : 0) | ((tp & 7) << 1) | ((rc & 1) << 4) |
                            ((dp & 7) << 5));
      if (tiled) codes[tiled_off(c, j, nch)] = v;
      else codes[(size_t)c * L + j] = v;
    }
  }
  hdr[c] = (uint64_t)(cf->mbs_log2 & 0xff) | ((uint64_t)(cf->p & 0xff) << 8);
}

/* device split: p powers of two summing to G, as even as possible (greedy doubling) */
static void split_devices(int p, int G, int *k) {
  int g[MAXP];
  for (int i = 0; i < p; ++i) g[i] = 1;
  int rem = G - p;
  while (rem > 0) {
    int best = -1;
    for (int i = 0; i < p; ++i)
      if (g[i] <= rem && (best < 0 || g[i] < g[best])) best = i;
    if (best < 0) break;
    rem -= g[best];
    g[best] *= 2;
  }
  for (int i = 0; i < p; ++i) k[i] = ilog2(g[i]);
}

/* keep the microbatch size within what the profile covers: dp <= mbs
   and per-GPU batch mbs/dp among the profiled sizes (n_b) */
static void fix_mbs(const gen_model *M, cfg_t *cf) {
  int need = 0, lo = 1 << 30;
  for (int i = 0; i < cf->p; ++i) {
    int d = cf->dpl[i];
    int d2 = d;
    if (cf->ft_from[i] < cf->start[i + 1]) d2 = d - cf->ft_d[i];
    int a = d < d2 ? d : d2, b = d < d2 ? d2 : d;
    if (b > need) need = b;
    if (a < lo) lo = a;
  }
  int cap = lo + M->n_b - 1;
  if (cf->mbs_log2 > cap) cf->mbs_log2 = cap;
  if (cf->mbs_log2 < need) cf->mbs_log2 = need;
}

static void base_config(const gen_model *M, uint64_t seed, int64_t group, cfg_t *cf) {
  rng_t r = rng_make(seed, 1, (uint64_t)group);
  int pmax = M->G < M->L ? M->G : M->L;
  if (pmax > MAXP) pmax = MAXP;
  /* stage count: powers of two favoured (parallel search over p) */
  int p;
  if (rng_below(&r, 4) != 0) {
    int kmax = ilog2(pmax);
    p = 1 << rng_below(&r, (uint32_t)(kmax + 1));
  } else {
    p = 1 + (int)rng_below(&r, (uint32_t)pmax);
  }
  cf->p = p;
  for (int i = 0; i <= p; ++i) cf->start[i] = (int)(((int64_t)M->L * i) / p); /* even partition */
  int k[MAXP];
  split_devices(p, M->G, k);
  /* a common data-parallel target keeps the per-GPU batch sizes of all stages
     inside the profiled range */
  int dstar = (int)rng_below(&r, (uint32_t)M->n_dp);
  for (int i = 0; i < p; ++i) {
    int dlo = k[i] - (M->n_tp - 1); if (dlo < 0) dlo = 0;
    int dhi = k[i] < M->n_dp - 1 ? k[i] : M->n_dp - 1;
    int d = dstar < dlo ? dlo : (dstar > dhi ? dhi : dstar);
    cf->dpl[i] = d;
    cf->tpl[i] = k[i] - d;
    cf->rcl[i] = 0;
    cf->ft_from[i] = M->L;
    cf->ft_d[i] = 0;
  }
  cf->mbs_log2 = 0;
  fix_mbs(M, cf); /* minimum microbatch size */
}

static void apply_primitive(const gen_model *M, cfg_t *cf, rng_t *r) {
  int p = cf->p;
  int log2Bg = ilog2(M->Bg);
  uint32_t kind = rng_below(r, 12);
  if (kind < 4) {
    /* inc/dec-op#: move the edge between stages i-1 and i */
    if (p < 2) return;
    int i = 1 + (int)rng_below(r, (uint32_t)(p - 1));
    int span = M->L / p / 4 + 1;
    int d = (int)rng_below(r, (uint32_t)(2 * span + 1)) - span;
    int s = cf->start[i] + d;
    if (s <= cf->start[i - 1]) s = cf->start[i - 1] + 1;
    if (s >= cf->start[i + 1]) s = cf->start[i + 1] - 1;
    if (s <= cf->start[i - 1] || s >= cf->start[i + 1]) return;
    cf->start[i] = s;
    for (int q = i - 1; q <= i; ++q)
      if (cf->ft_from[q] < cf->start[q]) cf->ft_from[q] = cf->start[q];
  } else if (kind < 5) {
    /* inc/dec-mbs (model level) */
    int d = rng_below(r, 2) ? 1 : -1;
    int m = cf->mbs_log2 + d;
    if (m < 0 || m > log2Bg) return;
    cf->mbs_log2 = m;
    fix_mbs(M, cf);
  } else if (kind < 7) {
    /* inc-dp / inc-tp on stage s with dec-dp/tp on a partner stage q.
       Device counts stay powers of two summing to G, so the partner must hold
       twice the devices of s: afterwards the two stages have swapped sizes. */
    if (p < 2) return;
    int s = (int)rng_below(r, (uint32_t)p);
    int ks = cf->tpl[s] + cf->dpl[s];
    int cand[MAXP], nc = 0;
    for (int q = 0; q < p; ++q)
      if (q != s && cf->tpl[q] + cf->dpl[q] == ks + 1) cand[nc++] = q;
    if (nc == 0) return;
    int q = cand[rng_below(r, (uint32_t)nc)];
    int use_tp = rng_below(r, 2);
    if (use_tp && cf->tpl[s] + 1 < M->n_tp) cf->tpl[s]++;
    else if (cf->dpl[s] + 1 < M->n_dp) cf->dpl[s]++;
    else if (cf->tpl[s] + 1 < M->n_tp) cf->tpl[s]++;
    else return;
    if (cf->dpl[q] > 0 && (rng_below(r, 2) || cf->tpl[q] == 0)) cf->dpl[q]--;
    else cf->tpl[q]--;
    cf->ft_from[s] = M->L;
    cf->ft_from[q] = M->L;
    fix_mbs(M, cf);
  } else if (kind < 8) {
    /* tp <-> dp trade inside stage s (inc-tp + dec-dp, same devices) */
    int s = (int)rng_below(r, (uint32_t)p);
    if (rng_below(r, 2)) {
      if (cf->dpl[s] > 0 && cf->tpl[s] + 1 < M->n_tp) { cf->tpl[s]++; cf->dpl[s]--; }
    } else {
      if (cf->tpl[s] > 0 && cf->dpl[s] + 1 < M->n_dp) { cf->tpl[s]--; cf->dpl[s]++; }
    }
    cf->ft_from[s] = M->L;
    fix_mbs(M, cf);
  } else if (kind < 11) {
    /* inc/dec-rc: greedy recompute of the largest-activation op types */
    int s = (int)rng_below(r, (uint32_t)p);
    int lv = cf->rcl[s] + (rng_below(r, 3) ? 1 : -1);
    if (lv < 0) lv = 0;
    if (lv > 4) lv = 4;
    cf->rcl[s] = lv == 4 ? 255 : lv;
  } else {
    /* op-level fine-tune: change tp/dp from op k to the end of the stage */
    int s = (int)rng_below(r, (uint32_t)p);
    int n = cf->start[s + 1] - cf->start[s];
    if (n < 2) return;
    int from = cf->start[s] + 1 + (int)rng_below(r, (uint32_t)(n - 1));
    int d = rng_below(r, 2) ? 1 : -1;
    int t2 = cf->tpl[s] + d, d2 = cf->dpl[s] - d;
    if (t2 < 0 || d2 < 0 || t2 >= M->n_tp || d2 >= M->n_dp) return;
    cf->ft_from[s] = from;
    cf->ft_d[s] = d;
    fix_mbs(M, cf);
  }
}

/* Search-shaped candidates [first, first+n) of a job; group_size candidates share a base. */
int gen_search_shaped(const gen_model *M, uint64_t seed, int64_t first, int64_t n,
                      int32_t group_size, int32_t invalid_permille, uint8_t *codes, int tiled,
                      uint64_t *hdr) {
  if (!M || M->L < 1 || M->G < 1 || n < 0 || group_size < 1) return -1;
  int nch = (M->L + 15) / 16;
  cfg_t base, cf;
  int64_t cur_group = -1;
  for (int64_t c = 0; c < n; ++c) {
    int64_t g = first + c;
    int64_t grp = g / group_size;
    if (grp != cur_group) { base_config(M, seed, grp, &base); cur_group = grp; }
    cf = base;
    rng_t r = rng_make(seed, 2, (uint64_t)g);
    int hops = 1 + (int)rng_below(&r, 7); /* MaxHops = 7 */
    for (int h = 0; h < hops; ++h) apply_primitive(M, &cf, &r);
    if (tiled) {
      for (int j = 0; j < nch * 16; ++j) codes[tiled_off(c, j, nch)] = 0;
    }
    emit(M, &cf, codes, hdr, c, tiled);
    if ((int32_t)rng_below(&r, 1000) < invalid_permille) {
      /* corrupt into an invalid encoding */
      uint32_t how = rng_below(&r, 4);
      size_t o0 = tiled ? tiled_off(c, 0, nch) : (size_t)c * M->L;
      if (how == 0) codes[o0] &= 0xFE;                           /* no head on op 0 */
      else if (how == 1) hdr[c] += 1ull << 8;                     /* p off by one */
      else if (how == 2) {                                        /* tp*dp mismatch in a stage */
        int j = (int)rng_below(&r, (uint32_t)M->L);
        size_t o = tiled ? tiled_off(c, j, nch) : (size_t)c * M->L + j;
        codes[o] ^= 0x02;
      } else hdr[c] = (hdr[c] & ~0xffull) | (uint64_t)(ilog2(M->Bg) + 1); /* mbs > Bg */
    }
  }
  return 0;
}

/* Dense-random (adversarial) candidates: valid stage structure, random per-op tp/dp mix and rc. */
int gen_dense_random(const gen_model *M, uint64_t seed, int64_t first, int64_t n, uint8_t *codes,
                     int tiled, uint64_t *hdr) {
  if (!M || M->L < 1 || M->G < 1 || n < 0) return -1;
  int L = M->L, nch = (L + 15) / 16;
  int pmax = M->G < L ? M->G : L;
  if (pmax > MAXP) pmax = MAXP;
  int *cut = (int *)malloc(sizeof(int) * (L + 1));
  for (int64_t c = 0; c < n; ++c) {
    rng_t r = rng_make(seed, 3, (uint64_t)(first + c));
    int p = 1 + (int)rng_below(&r, (uint32_t)pmax);
    /* p-1 distinct cut points in [1, L) by partial Fisher-Yates */
    int m = L - 1;
    for (int i = 0; i < m; ++i) cut[i] = i + 1;
    for (int i = 0; i < p - 1; ++i) {
      int k = i + (int)rng_below(&r, (uint32_t)(m - i));
      int t = cut[i]; cut[i] = cut[k]; cut[k] = t;
    }
    /* sort the first p-1 */
    for (int i = 1; i < p - 1; ++i) {
      int v = cut[i], k = i - 1;
      while (k >= 0 && cut[k] > v) { cut[k + 1] = cut[k]; k--; }
      cut[k + 1] = v;
    }
    int kdev[MAXP];
    split_devices(p, M->G, kdev);
    /* shuffle the device split across stages */
    for (int i = p - 1; i > 0; --i) {
      int k = (int)rng_below(&r, (uint32_t)(i + 1));
      int t = kdev[i]; kdev[i] = kdev[k]; kdev[k] = t;
    }
    int log2Bg = ilog2(M->Bg);
    int mb = (int)rng_below(&r, (uint32_t)(log2Bg + 1));
    if (tiled) for (int j = 0; j < nch * 16; ++j) codes[tiled_off(c, j, nch)] = 0;
    for (int i = 0; i < p; ++i) {
      int s0 = i == 0 ? 0 : cut[i - 1], s1 = i == p - 1 ? L : cut[i];
      int dlo = kdev[i] - (M->n_tp - 1); if (dlo < 0) dlo = 0;
      int dhi = kdev[i] < M->n_dp - 1 ? kdev[i] : M->n_dp - 1;
      /* per-GPU batch mbs/dp inside the profiled range when possible */
      int alo = dlo > mb - M->n_b + 1 ? dlo : mb - M->n_b + 1;
      int ahi = dhi < mb ? dhi : mb;
      if (alo > ahi) { alo = dlo; ahi = dhi; }
      for (int j = s0; j < s1; ++j) {
        int dp = alo + (int)rng_below(&r, (uint32_t)(ahi - alo + 1));
        int tp = kdev[i] - dp;
        int rc = (int)rng_below(&r, 2);
        uint8_t v = (uint8_t)((j == s0) | ((tp & 7) << 1) | (rc << 4) | ((dp & 7) << 5));
        if (tiled) codes[tiled_off(c, j, nch)] = v;
        else codes[(size_t)c * L + j] = v;
      }
    }
    hdr[c] = (uint64_t)(mb & 0xff) | ((uint64_t)p << 8);
  }
  free(cut);
  return 0;
}

/* ---- exhaustive enumeration of a tiny model -------------------------------
 * Order: mbs_log2 ascending; p ascending; stage cut vectors lexicographic;
 * per-stage log2 device counts (k_i, sum 2^k_i = G) lexicographic; then per op
 * (in op order, last op fastest): (tpl ascending, rc ascending) for per_op=1,
 * or per stage (tpl ascending) + per op rc for per_op=0 (stage-uniform tp/dp).
 * Returns the number of configurations; writes them if codes != NULL (row-major).
 */
typedef struct {
  const gen_model *M;
  int per_op;
  int64_t count, cap;
  uint8_t *codes;
  uint64_t *hdr;
  int mbs, p;
  int cut[MAXP + 1];
  int k[MAXP];
  uint8_t cur[64];
} enum_t;

static void enum_ops(enum_t *E, int j, int stage) {
  const gen_model *M = E->M;
  if (j == M->L) {
    if (E->codes && E->count < E->cap) {
      memcpy(E->codes + (size_t)E->count * M->L, E->cur, (size_t)M->L);
      E->hdr[E->count] = (uint64_t)E->mbs | ((uint64_t)E->p << 8);
    }
    E->count++;
    return;
  }
  int st = stage;
  if (st + 1 < E->p && j == E->cut[st + 1]) st++;
  int head = (j == E->cut[st]);
  int kk = E->k[st];
  int lo = kk - (M->n_dp - 1); if (lo < 0) lo = 0;
  int hi = kk < M->n_tp - 1 ? kk : M->n_tp - 1;
  if (!E->per_op && !head) {
    /* stage-uniform tp/dp: copy from the previous op of the stage */
    int tp = (E->cur[j - 1] >> 1) & 7, dp = (E->cur[j - 1] >> 5) & 7;
    for (int rc = 0; rc < 2; ++rc) {
      E->cur[j] = (uint8_t)(((tp & 7) << 1) | (rc << 4) | ((dp & 7) << 5));
      enum_ops(E, j + 1, st);
    }
    return;
  }
  for (int tp = lo; tp <= hi; ++tp) {
    int dp = kk - tp;
    for (int rc = 0; rc < 2; ++rc) {
      E->cur[j] = (uint8_t)(head | ((tp & 7) << 1) | (rc << 4) | ((dp & 7) << 5));
      enum_ops(E, j + 1, st);
    }
  }
}

static void enum_devices(enum_t *E, int i, int rem) {
  if (i == E->p) {
    if (rem == 0) enum_ops(E, 0, 0);
    return;
  }
  for (int kk = 0; (1 << kk) <= rem - (E->p - i - 1); ++kk) {
    int lo = kk - (E->M->n_dp - 1);
    if (lo > E->M->n_tp - 1) continue; /* no (tp, dp) for this device count */
    E->k[i] = kk;
    enum_devices(E, i + 1, rem - (1 << kk));
  }
}

static void enum_cuts(enum_t *E, int i) {
  const gen_model *M = E->M;
  if (i == E->p) {
    E->cut[E->p] = M->L;
    enum_devices(E, 0, M->G);
    return;
  }
  for (int c = E->cut[i - 1] + 1; c <= M->L - (E->p - i); ++c) {
    E->cut[i] = c;
    enum_cuts(E, i + 1);
  }
}

int64_t gen_exhaustive(const gen_model *M, int per_op, uint8_t *codes, uint64_t *hdr,
                       int64_t cap) {
  if (!M || M->L < 1 || M->L > 64) return -1;
  enum_t E;
  memset(&E, 0, sizeof(E));
  E.M = M;
  E.per_op = per_op;
  E.codes = codes;
  E.hdr = hdr;
  E.cap = cap;
  int log2Bg = ilog2(M->Bg);
  for (int mbs = 0; mbs <= log2Bg; ++mbs) {
    E.mbs = mbs;
    for (int p = 1; p <= M->G && p <= M->L; ++p) {
      E.p = p;
      E.cut[0] = 0;
      enum_cuts(&E, 1);
    }
  }
  return E.count;
}

/* Row-major -> tiled layout (host), pad bytes zero. */
void gen_tile(const uint8_t *rowmajor, int64_t n, int32_t L, uint8_t *tiled) {
  int nch = (L + 15) / 16;
  int64_t ntiles = (n + 31) / 32;
  memset(tiled, 0, (size_t)ntiles * nch * 512);
  for (int64_t c = 0; c < n; ++c)
    for (int j = 0; j < L; ++j) tiled[tiled_off(c, j, nch)] = rowmajor[(size_t)c * L + j];
}
