// aceso_capi.cu — the C-ABI of libaceso (include/aceso.h): profile validation and
// packing, launches of the sm_100a kernels, error reporting. No computation of
// the model happens on the host: every step of the evaluation path runs in the
// kernels of eval_kernel.cuh / aux_kernels.cuh.
#include <cuda_runtime.h>

#include <algorithm>
#include <array>
#include <map>
#include <cstdarg>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <string>
#include <vector>

#include "aux_kernels.cuh"
#include "common.cuh"
#include "dedup_kernels.cuh"
#include "expand_kernel.cuh"
#include "eval_kernel.cuh"
#include "event_kernel.cuh"
#include "dense_kernel.cuh"
#include "enum_kernel.cuh"
#include "scan_kernel.cuh"

using namespace aceso;

namespace {

thread_local std::string g_err;

int fail(int code, const char *fmt, ...) {
  char buf[512];
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(buf, sizeof(buf), fmt, ap);
  va_end(ap);
  g_err = buf;
  return code;
}

#define CUDA_TRY(expr)                                                                     \
  do {                                                                                     \
    cudaError_t e_ = (expr);                                                               \
    if (e_ != cudaSuccess)                                                                 \
      return fail(ACESO_ECUDA, "%s failed: %s", #expr, cudaGetErrorString(e_));            \
  } while (0)

// A pointer the kernels dereference must be device-accessible from `device`: its device memory,
// managed memory or mapped pinned host memory. Plain host memory (or another device's memory)
// would fault inside the kernel, a sticky error that ends the CUDA context, so it is refused
// here with ACESO_EINVAL naming the argument. Null is the caller's (size-dependent) check;
// device -1: any device (the context-free calls).
// The last 16 pointers that passed (exact addresses, with their device) are remembered per
// thread: loops that reuse their buffers every step query the driver once per buffer.
int check_dev_ptr(const void *p, const char *name, int device) {
  if (!p) return ACESO_OK;
  static thread_local const void *ok_ptr[16];
  static thread_local int ok_dev[16];
  static thread_local unsigned ok_next;
  for (int k = 0; k < 16; ++k)
    if (ok_ptr[k] == p && (device < 0 || ok_dev[k] == device)) return ACESO_OK;
  cudaPointerAttributes a;
  if (cudaPointerGetAttributes(&a, p) != cudaSuccess) {
    cudaGetLastError();  // clear the non-sticky lookup error
    return fail(ACESO_EINVAL, "%s: not a CUDA-visible pointer", name);
  }
  if (a.type == cudaMemoryTypeUnregistered) return fail(ACESO_EINVAL, "%s: host memory, not device-accessible", name);
  if (a.type == cudaMemoryTypeDevice && device >= 0 && a.device != device)
    return fail(ACESO_EINVAL, "%s: memory of device %d, context on device %d", name, a.device, device);
  if (device >= 0 || a.type == cudaMemoryTypeDevice) {  // remember it with the device it was checked for
    const unsigned k = ok_next++ & 15u;
    ok_ptr[k] = p;
    ok_dev[k] = device >= 0 ? device : a.device;
  }
  return ACESO_OK;
}
#define PTR_TRY(p, dev)                                       \
  do {                                                        \
    const int r_ = check_dev_ptr((p), #p, (dev));             \
    if (r_ != ACESO_OK) return r_;                            \
  } while (0)

template <int B>
void *quad_kernel_for(uint32_t mode) {
  switch (mode) {
    case 1: return reinterpret_cast<void *>(&eval_kernel<1, B>);
    case 2: return reinterpret_cast<void *>(&eval_kernel<2, B>);
    case 3: return reinterpret_cast<void *>(&eval_kernel<3, B>);
    case 4: return reinterpret_cast<void *>(&eval_kernel<4, B>);
    case 5: return reinterpret_cast<void *>(&eval_kernel<5, B>);
    case 6: return reinterpret_cast<void *>(&eval_kernel<6, B>);
    case 7: return reinterpret_cast<void *>(&eval_kernel<7, B>);
    default: return nullptr;
  }
}

template <int B, int W, int SC, bool OCT>
void *event_kernel_for(uint32_t mode) {
  switch (mode) {
    case 1: return reinterpret_cast<void *>(&event_kernel<1, B, W, SC, OCT>);
    case 2: return reinterpret_cast<void *>(&event_kernel<2, B, W, SC, OCT>);
    case 3: return reinterpret_cast<void *>(&event_kernel<3, B, W, SC, OCT>);
    case 4: return reinterpret_cast<void *>(&event_kernel<4, B, W, SC, OCT>);
    case 5: return reinterpret_cast<void *>(&event_kernel<5, B, W, SC, OCT>);
    case 6: return reinterpret_cast<void *>(&event_kernel<6, B, W, SC, OCT>);
    case 7: return reinterpret_cast<void *>(&event_kernel<7, B, W, SC, OCT>);
    default: return nullptr;
  }
}

// the event kernel's CTA shapes: (warps per CTA, register target in resident CTAs per SM).
// Built: 8 warps at 2 or 3 CTAs per SM. Measured and dropped (round 2, every BASELINE
// workload): 6 warps x 3 CTAs (18 warps per SM at 96 registers), 4 warps x 4 / 5 / 6 CTAs —
// within 0.3% of the better 8-warp shape on the 1K-layer model and 1-10% slower elsewhere.
// Ring slots: 8 chunks (4 KB) at 2 CTAs per SM (needs the octet tables), 4 chunks (2 KB)
// otherwise; octet recompute lookups whenever the octet tables exist.
void *event_kernel_shape(uint32_t mode, int warps, int minb, int sc, int oct) {
  (void)warps;
  if (minb == 2) {
    if (sc == 8) return event_kernel_for<2, 8, 8, true>(mode);
    return oct ? event_kernel_for<2, 8, 4, true>(mode) : event_kernel_for<2, 8, 4, false>(mode);
  }
  return oct ? event_kernel_for<3, 8, 4, true>(mode) : event_kernel_for<3, 8, 4, false>(mode);
}

template <int B>
void *dense_kernel_for(uint32_t mode) {
  switch (mode) {
    case 1: return reinterpret_cast<void *>(&dense_kernel<1, B>);
    case 2: return reinterpret_cast<void *>(&dense_kernel<2, B>);
    case 3: return reinterpret_cast<void *>(&dense_kernel<3, B>);
    case 4: return reinterpret_cast<void *>(&dense_kernel<4, B>);
    case 5: return reinterpret_cast<void *>(&dense_kernel<5, B>);
    case 6: return reinterpret_cast<void *>(&dense_kernel<6, B>);
    case 7: return reinterpret_cast<void *>(&dense_kernel<7, B>);
    default: return nullptr;
  }
}

template <bool GT>
void *dense_dims_kernel_for(uint32_t mode) {
  switch (mode) {
    case 1: return reinterpret_cast<void *>(&dense_kernel<1, 2, true, GT>);
    case 2: return reinterpret_cast<void *>(&dense_kernel<2, 2, true, GT>);
    case 3: return reinterpret_cast<void *>(&dense_kernel<3, 2, true, GT>);
    case 4: return reinterpret_cast<void *>(&dense_kernel<4, 2, true, GT>);
    case 5: return reinterpret_cast<void *>(&dense_kernel<5, 2, true, GT>);
    case 6: return reinterpret_cast<void *>(&dense_kernel<6, 2, true, GT>);
    case 7: return reinterpret_cast<void *>(&dense_kernel<7, 2, true, GT>);
    default: return nullptr;
  }
}

template <bool E64, int B>
void *scan_kernel_for(uint32_t mode) {
  switch (mode) {
    case 1: return reinterpret_cast<void *>(&scan_kernel<1, E64, B>);
    case 2: return reinterpret_cast<void *>(&scan_kernel<2, E64, B>);
    case 3: return reinterpret_cast<void *>(&scan_kernel<3, E64, B>);
    case 4: return reinterpret_cast<void *>(&scan_kernel<4, E64, B>);
    case 5: return reinterpret_cast<void *>(&scan_kernel<5, E64, B>);
    case 6: return reinterpret_cast<void *>(&scan_kernel<6, E64, B>);
    case 7: return reinterpret_cast<void *>(&scan_kernel<7, E64, B>);
    default: return nullptr;
  }
}

// kernel 0: per-op/quad kernel (eval_kernel.cuh); kernel 1: event kernel (event_kernel.cuh);
// kernel 2: dense kernel (dense_kernel.cuh, ACESO_HINT_DENSE); kernel 3: scan kernel
// (scan_kernel.cuh, exact u64 tables; e64: wide transient-memory table)
void *eval_kernel_for(uint32_t mode, int minb, int kernel, int e64 = 0, int ev_warps = kWarps, int ev_sc = 4,
                      int ev_oct = 0) {
  if (kernel == 3) {
    // the scan kernel's default register target is 2 CTAs per SM (its ring and lists take
    // ~100 KB of shared memory per CTA); ACESO_MINB=3 selects the 80-register build
    if (minb == 3 && getenv("ACESO_MINB")) return e64 ? scan_kernel_for<true, 3>(mode) : scan_kernel_for<false, 3>(mode);
    return e64 ? scan_kernel_for<true, 2>(mode) : scan_kernel_for<false, 2>(mode);
  }
  if (kernel == 1) return event_kernel_shape(mode, ev_warps, minb, ev_sc, ev_oct);
  if (kernel == 2) return minb == 2 ? dense_kernel_for<2>(mode) : dense_kernel_for<3>(mode);
  return minb == 2 ? quad_kernel_for<2>(mode) : quad_kernel_for<3>(mode);
}

uint32_t bitlen(uint64_t v) {
  uint32_t b = 0;
  while (v) { b++; v >>= 1; }
  return b;
}

}  // namespace

struct aceso_ctx {
  int device;
  int sms;
  int32_t L, T, n_tp, n_dp, n_b, G;
  uint64_t Bg, C;
  uint32_t mem_shift;
  Tables tab;
  void *d_blob;
  int kernel;       // default schedule: 0 per-op (quad) kernel, 1 event kernel (ACESO_KERNEL=quad|events)
  int quad_ok;      // the per-op kernel's tables fit in shared memory
  void *d_ev;       // event-kernel tables
  uint32_t qo_off, qo_bytes;
  const uint4 *px, *kx, *qr;
  const uint4 *qr8;      // octet recompute records (8-chunk slots), null without them
  const uint32_t *qo8;   // octet signature offsets
  const uint64_t *pd;
  const uint32_t *st;
  int minb;         // register target: 2 or 3 resident CTAs per SM
  int ev_warps;     // event kernel: warps per CTA (its kernels are templated on it; 8 is built)
  int ev_minb;      // event kernel: register target
  int ev_sc;        // event kernel: 16-op chunks per ring slot (8 at 2 CTAs per SM, else 4)
  int has_oct;      // octet recompute tables built (the 8-chunk-slot kernel needs them)
  int ev_oct;       // event kernel: octet recompute lookups (has_oct; ACESO_EV_OCT=0 turns them off)
  int tiles_per_warp;  // ACESO_TILES_PER_WARP (measurement knob): tiles each warp walks per launch (default 1)
  int max_ctas[4][8];  // per kernel and mode: resident CTAs (occupancy x SMs)
  int dense_kernel;    // schedule of ACESO_HINT_DENSE: 2 dense kernel (default), 0 per-op kernel (ACESO_DENSE_KERNEL=quad)
  size_t smem[4][8];
  int packed_ok;       // memory values fit the 32-bit packed tables of kernels 0-2 (else: scan kernel only)
  void *d_sc;          // scan-kernel tables
  const uint4 *sx, *sk, *sq;
  const uint64_t *sd;
  const void *ss;
  const uint32_t *sqo;
  uint32_t qo_words, es;
  int e64;             // scan kernel: transient-memory table in u64 (values >= 2^32 units)
  uint32_t sc_resolve; // scan kernel: resolve recompute-only chunks in the compacted pass (ACESO_SCAN_NORESOLVE=1: in the walk)
  int has_alt;         // alternative-dimension records loaded (aceso_eval_dims)
  int dims_gt;         // aceso_eval_dims: dense tables in global memory (too large for shared memory)
  size_t dims_smem[8];
  int dims_max_ctas[8];
};

// chunks per ring slot of the event kernel in this mode: FULL keeps 4 (its 16-byte list records
// would not leave room for two 8-chunk CTAs per SM)
static int ev_sc_for(const aceso_ctx *ctx, uint32_t mode) { return (mode & ACESO_OUT_FULL) ? 4 : ctx->ev_sc; }


namespace {
// kernel parameter block of a call (tables, outputs, selection); codes/hdr set by the caller
EvalParams make_params(const aceso_ctx *ctx, int64_t n, int64_t global_offset, int64_t n_total,
                       const aceso_eval_out *out, void *d_sel) {
  EvalParams P;
  memset(&P, 0, sizeof(P));
  P.n = n;
  P.gofs = global_offset;
  P.n_tiles = (n + 31) / 32;
  P.L = ctx->L;
  P.nch = (ctx->L + 15) / 16;
  P.T = ctx->T;
  P.n_tp = ctx->n_tp;
  P.n_dp = ctx->n_dp;
  P.n_b = ctx->n_b;
  P.G = ctx->G;
  P.Bg = ctx->Bg;
  P.C = ctx->C;
  P.mem_shift = ctx->mem_shift;
  P.blob = reinterpret_cast<const uint4 *>(ctx->d_blob);
  P.tab = ctx->tab;
  if (out) {
    P.iter_ns = out->iter_ns;
    P.max_mem = out->max_mem;
    P.info = out->info;
    P.stage_T = out->stage_T;
    P.stage_mem = out->stage_mem;
    P.stage_comp = out->stage_comp;
    P.stage_comm = out->stage_comm;
    P.p_max = out->p_max;
  }
  P.sel = reinterpret_cast<unsigned char *>(d_sel);
  P.n_total = n_total;
  P.ib = std::max(1u, bitlen((uint64_t)n_total));
  P.px = ctx->px;
  P.kx = ctx->kx;
  P.pd = ctx->pd;
  P.st = ctx->st;
  P.qr = ctx->qr;
  P.qr8 = ctx->qr8;
  P.qo8 = ctx->qo8;
  P.runs = (uint32_t)(ctx->n_b * ctx->n_tp);
  P.qo_bytes = ctx->qo_bytes;
  P.qo_off = ctx->qo_off;
  P.evblob = reinterpret_cast<const unsigned char *>(ctx->d_ev);
  P.sx = ctx->sx;
  P.sk = ctx->sk;
  P.sd = ctx->sd;
  P.ss = ctx->ss;
  P.sq = ctx->sq;
  P.sqo = ctx->sqo;
  P.qo_words = ctx->qo_words;
  P.es = ctx->es;
  P.sc_resolve = ctx->sc_resolve;
  P.n_minus = 1;
  return P;
}
}  // namespace

extern "C" {

const char *aceso_last_error(void) { return g_err.c_str(); }
const char *aceso_version(void) { return "aceso-b200 0.1 (sm_100a)"; }

size_t aceso_tiled_bytes(int64_t n, int32_t n_ops) {
  if (n < 0 || n_ops < 1) return 0;
  return (size_t)((n + 31) / 32) * (size_t)((n_ops + 15) / 16) * 512;
}

int aceso_load_profile(const aceso_profile_desc *d, int cuda_device, aceso_ctx **out) {
  if (!d || !out) return fail(ACESO_EINVAL, "null argument");
  *out = nullptr;
  if (d->n_ops < 1 || d->n_ops > kMaxOps) return fail(ACESO_EINVAL, "n_ops %d outside [1, %d]", d->n_ops, kMaxOps);
  if (d->n_types < 1 || d->n_types > 4096) return fail(ACESO_EINVAL, "n_types %d outside [1, 4096]", d->n_types);
  if (d->n_tp < 1 || d->n_tp > 8 || d->n_dp < 1 || d->n_dp > 8)
    return fail(ACESO_EINVAL, "n_tp/n_dp must be in [1, 8]");
  if (d->n_b < 1 || d->n_b > 16) return fail(ACESO_EINVAL, "n_b %d outside [1, 16]", d->n_b);
  if (d->n_devices < 1 || d->n_devices > 255) return fail(ACESO_EINVAL, "n_devices outside [1, 255]");
  if (d->global_batch < 1 || d->global_batch > (1ll << 31)) return fail(ACESO_EINVAL, "global_batch outside [1, 2^31]");
  if (d->mem_capacity < 0) return fail(ACESO_EINVAL, "negative mem_capacity");
  if (!d->op_type || !d->rec || !d->wmem || !d->dps) return fail(ACESO_EINVAL, "null table");
  const int L = d->n_ops, T = d->n_types, NT = d->n_tp, ND = d->n_dp, NB = d->n_b;
  for (int j = 0; j < L; ++j)
    if (d->op_type[j] >= T) return fail(ACESO_EINVAL, "op_type[%d] = %d >= n_types", j, d->op_type[j]);

  const uint64_t U32 = 0xffffffffull;
  const int n_alt = d->rec_alt ? 2 : 1;  // record sets: default dimension (+ the alternative)
  auto RA = [&](int alt, int t, int tp, int b, int f) {
    return (alt ? d->rec_alt : d->rec)[(((int64_t)t * NT + tp) * NB + b) * ACESO_REC_FIELDS + f];
  };
  auto R = [&](int t, int tp, int b, int f) { return RA(0, t, tp, b, f); };
  uint64_t maxSop = 0, maxRes = 0, maxP2P = 0, maxA = 0, maxE = 0, maxW = 0, maxD = 0;
  for (int t = 0; t < T; ++t)
    for (int tp = 0; tp < NT; ++tp) {
      for (int alt = 0; alt < n_alt; ++alt)
      for (int b = 0; b < NB; ++b) {
        for (int f = 0; f < ACESO_REC_FIELDS; ++f) {
          int64_t v = RA(alt, t, tp, b, f);
          const bool memf = (f == ACESO_F_ACT || f == ACESO_F_KEEP || f == ACESO_F_PEAK);
          if (v < 0 || (uint64_t)v > (memf ? (1ull << 40) : U32))
            return fail(ACESO_ERANGE, "%s[%d][%d][%d][%d] = %lld out of range", alt ? "rec_alt" : "rec", t, tp, b,
                        f, (long long)v);
        }
        uint64_t fc = RA(alt, t, tp, b, 0), fm = RA(alt, t, tp, b, 1), bc = RA(alt, t, tp, b, 2), bm = RA(alt, t, tp, b, 3);
        uint64_t act = RA(alt, t, tp, b, 4), keep = RA(alt, t, tp, b, 5), peak = RA(alt, t, tp, b, 6);
        if (keep > act) return fail(ACESO_ERANGE, "keep > act at %s[%d][%d][%d]", alt ? "rec_alt" : "rec", t, tp, b);
        uint64_t s1 = 2 * (fc + fm) + bc + bm;
        uint64_t e1 = peak + act - keep;
        maxSop = std::max(maxSop, s1);
        maxRes = std::max(maxRes, (uint64_t)RA(alt, t, tp, b, 7));
        maxP2P = std::max(maxP2P, (uint64_t)std::max(RA(alt, t, tp, b, 8), RA(alt, t, tp, b, 9)));
        maxA = std::max(maxA, act);
        maxE = std::max(maxE, e1);
      }
      int64_t pg = d->wmem[((int64_t)t * NT + tp) * 2], op = d->wmem[((int64_t)t * NT + tp) * 2 + 1];
      if (pg < 0 || op < 0 || pg > (1ll << 40) || op > (1ll << 40)) return fail(ACESO_ERANGE, "wmem[%d][%d] not in [0, 2^40]", t, tp);
      maxW = std::max(maxW, (uint64_t)(pg + op));
      for (int dp = 0; dp < ND; ++dp) {
        int64_t v = d->dps[((int64_t)t * NT + tp) * ND + dp];
        if (v < 0 || (uint64_t)v > U32) return fail(ACESO_ERANGE, "dps[%d][%d][%d] not in [0, 2^32)", t, tp, dp);
        maxD = std::max(maxD, (uint64_t)v);
      }
    }
  // memory fields are packed in units of 2^ms bytes (exact): ms = common trailing zeros
  uint32_t ms = 16;
  {
    auto tz = [&](int64_t v) { if (v != 0) ms = std::min<uint32_t>(ms, (uint32_t)__builtin_ctzll((uint64_t)v)); };
    for (int t = 0; t < T; ++t)
      for (int tp = 0; tp < NT; ++tp) {
        for (int alt = 0; alt < n_alt; ++alt)
          for (int b = 0; b < NB; ++b) { tz(RA(alt, t, tp, b, 4)); tz(RA(alt, t, tp, b, 5)); tz(RA(alt, t, tp, b, 6)); }
        tz(d->wmem[((int64_t)t * NT + tp) * 2]);
        tz(d->wmem[((int64_t)t * NT + tp) * 2 + 1]);
      }
  }
  // the packed kernels (per-op, event v2, dense) hold per-op values in 32-bit fields: memory in
  // units of 2^ms bytes, recomputed op times in ns; the scan kernel is exact for every profile
  const bool packed_ok = (maxA >> ms) <= U32 && (maxE >> ms) <= U32 && (maxW >> ms) <= U32 && maxSop <= U32;
  {
    // model-wide bounds: every iteration time / stage memory < 2^62 (exact keys)
    typedef unsigned __int128 u128;
    const u128 lim = (u128)1 << 62;
    u128 tb = ((u128)L * (maxSop + maxRes + maxD) + (u128)2 * d->n_devices * maxP2P) * ((u128)d->global_batch + 1);
    u128 mb = (u128)L * maxW + (u128)d->global_batch * L * maxA + maxE;
    if (tb >= lim) return fail(ACESO_ERANGE, "iteration-time bound exceeds 2^62");
    if (mb >= lim) return fail(ACESO_ERANGE, "memory bound exceeds 2^62");
  }

  // ---- pack tables ----
  const uint32_t S = kTypeStride;
  const uint32_t RUNS = (uint32_t)NB * NT;
  const int nch = (L + 15) / 16;
  const int nquads = nch * 4;  // quads incl. the zero-padded tail
  auto a16 = [](uint32_t v) { return (v + 15u) & ~15u; };
  // quad signatures: distinct type 4-tuples of the full quads
  std::vector<int> qsig(nquads, -1);
  std::vector<std::array<uint16_t, 4>> sigs;
  {
    std::map<std::array<uint16_t, 4>, int> seen;
    for (int q = 0; q < nquads; ++q) {
      if (4 * q + 4 > L) continue;
      std::array<uint16_t, 4> key = {d->op_type[4 * q], d->op_type[4 * q + 1], d->op_type[4 * q + 2], d->op_type[4 * q + 3]};
      auto it = seen.find(key);
      if (it == seen.end()) {
        it = seen.emplace(key, (int)sigs.size()).first;
        sigs.push_back(key);
      }
      qsig[q] = it->second;
    }
  }
  const uint32_t NS = (uint32_t)sigs.size();
  const uint32_t bytesR = RUNS * T * S;
  const uint32_t bytesD = (uint32_t)NT * T * S;
  const uint32_t bytesT = a16((uint32_t)nch * 16 * 2);
  const uint32_t bytesQO = (uint32_t)nquads * 8;
  const uint32_t bytesQT = NS * RUNS * 32;
  const uint32_t bytesQD = NS * (uint32_t)NT * 32;
  const uint32_t bytesF = a16(RUNS * T * 8);
  const uint32_t bytesQF = a16(NS * RUNS * 8);
  const uint32_t bytesK = RUNS * T * 16;
  Tables tab;
  memset(&tab, 0, sizeof(tab));
  tab.offR = 0;
  tab.offD = tab.offR + bytesR;
  tab.offT = tab.offD + bytesD;
  tab.offQO = tab.offT + bytesT;
  tab.offQT = tab.offQO + bytesQO;
  tab.offQD = tab.offQT + bytesQT;
  tab.bytes = tab.offQD + bytesQD;
  tab.offF = tab.bytes;
  tab.offQF = tab.offF + bytesF;
  tab.bytes_full = tab.offQF + bytesQF;
  tab.offK = tab.bytes_full;
  tab.bytesK = bytesK;
  // stage the cold table too when shared memory allows ~2 CTAs per SM
  tab.k_smem = (tab.bytes_full + bytesK + kRingBytesPerCta + 16384u <= 100u * 1024u) ? 1u : 0u;
  // the per-op kernel stages its tables in shared memory; larger profiles use the event
  // kernel only (its tables are in global memory)
  const bool quad_ok = tab.bytes_full + kRingBytesPerCta + 16384u <= 220u * 1024u;
  // dense-kernel tables: 2T types when alternative-dimension records are given (type + T)
  const uint32_t T2 = (uint32_t)(n_alt * T);
  tab.dOff = a16(tab.offK + bytesK);
  tab.dR = 0;
  tab.dD = tab.dR + RUNS * T2 * S;
  tab.dK = tab.dD + (uint32_t)NT * T2 * S;
  tab.dT = tab.dK + RUNS * T2 * 16;
  tab.dbytes = tab.dT + bytesT;
  tab.dF = tab.dbytes;
  tab.dbytes_full = tab.dF + a16(RUNS * T2 * 8);
  const bool dense_ok = tab.dbytes_full + kRingBytesPerCta + 16384u <= 220u * 1024u;
  const uint32_t blob_bytes = tab.dOff + tab.dbytes_full;
  std::vector<uint32_t> blob(blob_bytes / 4, 0u);
  auto rec_S = [&](int t, int tp, int b, int rc) -> uint64_t {
    uint64_t F = (uint64_t)R(t, tp, b, 0) + R(t, tp, b, 1);
    return F + R(t, tp, b, 2) + R(t, tp, b, 3) + (rc ? F : 0);
  };
  auto rec_A = [&](int t, int tp, int b, int rc) -> uint64_t { return (uint64_t)(rc ? R(t, tp, b, 5) : R(t, tp, b, 4)) >> ms; };
  auto rec_e = [&](int t, int tp, int b, int rc) -> uint64_t {
    return ((uint64_t)R(t, tp, b, 6) + (rc ? (uint64_t)(R(t, tp, b, 4) - R(t, tp, b, 5)) : 0)) >> ms;
  };
  auto rec_W = [&](int t, int tp) -> uint64_t {
    return ((uint64_t)d->wmem[((int64_t)t * NT + tp) * 2] + (uint64_t)d->wmem[((int64_t)t * NT + tp) * 2 + 1]) >> ms;
  };
  auto rec_C = [&](int t, int tp, int b, int rc) -> uint64_t {
    return (uint64_t)R(t, tp, b, 0) + R(t, tp, b, 2) + (rc ? (uint64_t)R(t, tp, b, 0) : 0);
  };
  auto dps_of = [&](int t, int tp, int dp) -> uint64_t { return (uint64_t)d->dps[((int64_t)t * NT + tp) * ND + dp]; };
  for (int b = 0; b < NB; ++b)
    for (int tp = 0; tp < NT; ++tp)
      for (int t = 0; t < T; ++t) {
        const uint32_t rt = (uint32_t)(b * NT + tp) * T + t;  // (run, type) index
        for (int rc = 0; rc < 2; ++rc) {
          uint32_t *r = &blob[(tab.offR / 4) + rt * (S / 4) + rc * 4];
          r[0] = (uint32_t)rec_S(t, tp, b, rc);
          r[1] = (uint32_t)rec_A(t, tp, b, rc);
          r[2] = (uint32_t)rec_e(t, tp, b, rc);
          r[3] = (uint32_t)rec_W(t, tp);
          blob[(tab.offF / 4) + rt * 2 + rc] = (uint32_t)rec_C(t, tp, b, rc);
        }
        uint32_t *k = &blob[(tab.offK / 4) + rt * 4];
        k[0] = (uint32_t)R(t, tp, b, 7);
        k[1] = (uint32_t)R(t, tp, b, 8);
        k[2] = (uint32_t)R(t, tp, b, 9);
      }
  // dense-kernel copies, type-major; types T..2T-1: the alternative dimension's records (same
  // parameter bytes and DP sync: the partition dimension does not change the weights per GPU)
  for (uint32_t t2 = 0; t2 < T2; ++t2)
    for (int b = 0; b < NB; ++b)
      for (int tp = 0; tp < NT; ++tp) {
        const int t = (int)(t2 % (uint32_t)T), alt = t2 >= (uint32_t)T;
        auto F = [&](int f) { return (uint64_t)RA(alt, t, tp, b, f); };
        const uint32_t tr = t2 * RUNS + (uint32_t)(b * NT + tp);  // (type, run) index
        for (int rc = 0; rc < 2; ++rc) {
          const uint64_t Fw = F(0) + F(1);
          uint32_t *r = &blob[(tab.dOff + tab.dR) / 4 + tr * 8 + rc * 4];
          r[0] = (uint32_t)(Fw + F(2) + F(3) + (rc ? Fw : 0));
          r[1] = (uint32_t)((rc ? F(5) : F(4)) >> ms);
          r[2] = (uint32_t)((F(6) + (rc ? F(4) - F(5) : 0)) >> ms);
          r[3] = (uint32_t)rec_W(t, tp);
          blob[(tab.dOff + tab.dF) / 4 + tr * 2 + rc] = (uint32_t)(F(0) + F(2) + (rc ? F(0) : 0));
        }
        uint32_t *dk = &blob[(tab.dOff + tab.dK) / 4 + tr * 4];
        dk[0] = (uint32_t)F(7);
        dk[1] = (uint32_t)F(8);
        dk[2] = (uint32_t)F(9);
      }
  for (int tp = 0; tp < NT; ++tp)
    for (int t = 0; t < T; ++t)
      for (int dp = 0; dp < ND; ++dp) {
        blob[(tab.offD + ((uint32_t)tp * T + t) * S) / 4 + dp] = (uint32_t)dps_of(t, tp, dp);
        for (int alt = 0; alt < n_alt; ++alt)
          blob[(tab.dOff + tab.dD) / 4 + (((uint32_t)(t + alt * T)) * NT + tp) * 8 + dp] = (uint32_t)dps_of(t, tp, dp);
      }
  {
    uint16_t *tt = reinterpret_cast<uint16_t *>(&blob[tab.offT / 4]);
    uint16_t *dt = reinterpret_cast<uint16_t *>(&blob[(tab.dOff + tab.dT) / 4]);
    for (int j = 0; j < L; ++j) tt[j] = dt[j] = d->op_type[j];
  }
  // quad sums; a signature whose sums do not fit 32 bits is not used (per-op path)
  std::vector<char> sig_ok(NS, 1);
  for (uint32_t sg = 0; sg < NS; ++sg) {
    const auto &ty = sigs[sg];
    for (int b = 0; b < NB; ++b)
      for (int tp = 0; tp < NT; ++tp) {
        const uint32_t run = (uint32_t)(b * NT + tp);
        for (int rc = 0; rc < 2; ++rc) {
          uint64_t sS = 0, sA = 0, mE = 0, sW = 0, sC = 0;
          for (int k = 0; k < 4; ++k) {
            sS += rec_S(ty[k], tp, b, rc);
            sA += rec_A(ty[k], tp, b, rc);
            mE = std::max(mE, rec_e(ty[k], tp, b, rc));
            sW += rec_W(ty[k], tp);
            sC += rec_C(ty[k], tp, b, rc);
          }
          if (sS > U32 || sA > U32 || sW > U32 || sC > U32) sig_ok[sg] = 0;
          uint32_t *q = &blob[(tab.offQT / 4) + (sg * RUNS + run) * 8 + rc * 4];
          q[0] = (uint32_t)sS; q[1] = (uint32_t)sA; q[2] = (uint32_t)mE; q[3] = (uint32_t)sW;
          blob[(tab.offQF / 4) + (sg * RUNS + run) * 2 + rc] = (uint32_t)sC;
        }
      }
    for (int tp = 0; tp < NT; ++tp)
      for (int dp = 0; dp < ND; ++dp) {
        uint64_t sD = 0;
        for (int k = 0; k < 4; ++k) sD += dps_of(ty[k], tp, dp);
        if (sD > U32) sig_ok[sg] = 0;
        blob[(tab.offQD / 4) + (sg * NT + tp) * 8 + dp] = (uint32_t)sD;
      }
  }
  for (int q = 0; q < nquads; ++q) {
    uint32_t *o = &blob[(tab.offQO / 4) + q * 2];
    if (qsig[q] >= 0 && sig_ok[qsig[q]]) {
      o[0] = (uint32_t)qsig[q] * RUNS * 32;
      o[1] = (uint32_t)qsig[q] * NT * 32;
    } else {
      o[0] = 0xffffffffu;
      o[1] = 0;
    }
  }

  // ---- event-kernel tables (event_kernel.cuh): position prefixes per run ----
  const uint32_t Lp1 = (uint32_t)L + 1u;
  const int levels = 32 - __builtin_clz((unsigned)L);  // floor(log2 L) + 1
  const int nq = (L + 3) / 4;
  std::vector<uint32_t> eqo(nq);
  std::vector<std::array<int, 4>> esigs;
  {
    std::map<std::array<int, 4>, int> seen;
    for (int q = 0; q < nq; ++q) {
      std::array<int, 4> key;
      for (int k = 0; k < 4; ++k) key[k] = 4 * q + k < L ? (int)d->op_type[4 * q + k] : -1;
      auto it = seen.find(key);
      if (it == seen.end()) {
        it = seen.emplace(key, (int)esigs.size()).first;
        esigs.push_back(key);
      }
      eqo[q] = (uint32_t)it->second * RUNS * 16u;
    }
  }
  // octet signatures (distinct type 8-tuples at ops 8o..8o+7): the 8-chunk-slot event kernel
  // looks up a recompute-only chunk's deltas per octet (256 patterns) instead of per quad
  const int no8 = 2 * ((L + 15) / 16);
  std::vector<uint32_t> eo8(no8);
  std::vector<std::array<int, 8>> osigs;
  {
    std::map<std::array<int, 8>, int> seen;
    for (int o = 0; o < no8; ++o) {
      std::array<int, 8> key;
      for (int k = 0; k < 8; ++k) key[k] = 8 * o + k < L ? (int)d->op_type[8 * o + k] : -1;
      auto it = seen.find(key);
      if (it == seen.end()) {
        it = seen.emplace(key, (int)osigs.size()).first;
        osigs.push_back(key);
      }
      eo8[o] = (uint32_t)it->second * RUNS * 256u;
    }
  }
  // octet table budget: at most 64 MB (else the quad tables serve every schedule)
  const bool has_oct = osigs.size() * (size_t)RUNS * 256 * 32 <= ((size_t)64 << 20);
  auto al = [](size_t v) { return (v + 255) & ~(size_t)255; };
  const size_t ev_px = 0;
  const size_t ev_kx = al(ev_px + (size_t)RUNS * Lp1 * 32);
  const size_t ev_pd = al(ev_kx + (size_t)RUNS * Lp1 * 16);
  const size_t ev_st = al(ev_pd + (size_t)NT * ND * Lp1 * 8);
  const size_t ev_qr = al(ev_st + (size_t)levels * RUNS * L * 4);
  const size_t ev_qo = al(ev_qr + esigs.size() * RUNS * 16 * 32);
  const uint32_t qo_bytes = a16((uint32_t)nq * 4u);
  const size_t ev_qo8 = al(ev_qo + qo_bytes);
  const size_t ev_qr8 = al(ev_qo8 + (size_t)no8 * 4);
  const size_t ev_bytes = has_oct ? al(ev_qr8 + osigs.size() * RUNS * 256 * 32) : al(ev_qo + qo_bytes);
  std::vector<unsigned char> ev(ev_bytes, 0);
  {
    auto put64 = [&](size_t off, uint64_t v) { memcpy(&ev[off], &v, 8); };
    auto put32 = [&](size_t off, uint32_t v) { memcpy(&ev[off], &v, 4); };
    for (int b = 0; b < NB; ++b)
      for (int tp = 0; tp < NT; ++tp) {
        const uint32_t rr = (uint32_t)(b * NT + tp);
        uint64_t PS = 0, PA = 0, PW = 0, PC = 0;
        for (uint32_t j = 0; j <= (uint32_t)L; ++j) {
          const size_t o = (size_t)rr * Lp1 + j;
          put64(ev_px + o * 32, PS);
          put64(ev_px + o * 32 + 8, PA);
          put64(ev_px + o * 32 + 16, PW);
          put64(ev_px + o * 32 + 24, PC);
          if (j < (uint32_t)L) {
            const int t = d->op_type[j];
            PS += rec_S(t, tp, b, 0);
            PA += rec_A(t, tp, b, 0);
            PW += rec_W(t, tp);
            PC += rec_C(t, tp, b, 0);
            put32(ev_kx + o * 16, (uint32_t)R(t, tp, b, ACESO_F_RESHARD));
            put32(ev_kx + o * 16 + 4, (uint32_t)R(t, tp, b, ACESO_F_P2P_BWD));
            put32(ev_st + ((size_t)rr * L + j) * 4, (uint32_t)rec_e(t, tp, b, 0));
          }
          if (j > 0) put32(ev_kx + o * 16 + 8, (uint32_t)R(d->op_type[j - 1], tp, b, ACESO_F_P2P_FWD));
        }
        for (int k = 1; k < levels; ++k)
          for (int j = 0; j < L; ++j) {
            const int j2 = std::min(j + (1 << (k - 1)), L - 1);
            uint32_t v1, v2;
            memcpy(&v1, &ev[ev_st + (((size_t)(k - 1) * RUNS + rr) * L + j) * 4], 4);
            memcpy(&v2, &ev[ev_st + (((size_t)(k - 1) * RUNS + rr) * L + j2) * 4], 4);
            put32(ev_st + (((size_t)k * RUNS + rr) * L + j) * 4, std::max(v1, v2));
          }
        for (size_t sg = 0; sg < esigs.size(); ++sg)
          for (uint32_t m = 1; m < 16; ++m) {
            uint64_t dS = 0, dA = 0, dC = 0, E1 = 0;
            for (int k = 0; k < 4; ++k) {
              const int t = esigs[sg][k];
              if (t < 0 || !((m >> k) & 1u)) continue;
              dS += (uint64_t)R(t, tp, b, ACESO_F_FWD_COMP) + R(t, tp, b, ACESO_F_FWD_COMM);
              dA += (uint64_t)(R(t, tp, b, ACESO_F_ACT) - R(t, tp, b, ACESO_F_KEEP)) >> ms;
              dC += (uint64_t)R(t, tp, b, ACESO_F_FWD_COMP);
              E1 = std::max(E1, rec_e(t, tp, b, 1));
            }
            const size_t o = ev_qr + (((size_t)sg * RUNS + rr) * 16 + m) * 32;
            put64(o, dS);
            put64(o + 8, dA);
            put32(o + 16, (uint32_t)E1);
            put64(o + 24, dC);
          }
      }
    if (has_oct) {
      for (int o = 0; o < no8; ++o) put32(ev_qo8 + (size_t)o * 4, eo8[o]);
      for (int b = 0; b < NB; ++b)
        for (int tp = 0; tp < NT; ++tp) {
          const uint32_t rr = (uint32_t)(b * NT + tp);
          for (size_t sg = 0; sg < osigs.size(); ++sg)
            for (uint32_t m = 1; m < 256; ++m) {
              uint64_t dS = 0, dA = 0, dC = 0, E1 = 0;
              for (int k = 0; k < 8; ++k) {
                const int t = osigs[sg][k];
                if (t < 0 || !((m >> k) & 1u)) continue;
                dS += (uint64_t)R(t, tp, b, ACESO_F_FWD_COMP) + R(t, tp, b, ACESO_F_FWD_COMM);
                dA += (uint64_t)(R(t, tp, b, ACESO_F_ACT) - R(t, tp, b, ACESO_F_KEEP)) >> ms;
                dC += (uint64_t)R(t, tp, b, ACESO_F_FWD_COMP);
                E1 = std::max(E1, rec_e(t, tp, b, 1));
              }
              const size_t o = ev_qr8 + (((size_t)sg * RUNS + rr) * 256 + m) * 32;
              put64(o, dS);
              put64(o + 8, dA);
              put32(o + 16, (uint32_t)E1);
              put64(o + 24, dC);
            }
        }
    }
    for (int tp = 0; tp < NT; ++tp)
      for (int dp = 0; dp < ND; ++dp) {
        uint64_t s = 0;
        for (uint32_t j = 0; j <= (uint32_t)L; ++j) {
          put64(ev_pd + (((size_t)tp * ND + dp) * Lp1 + j) * 8, s);
          if (j < (uint32_t)L) s += dps_of(d->op_type[j], tp, dp);
        }
      }
    for (int q = 0; q < nq; ++q) put32(ev_qo + (size_t)q * 4, eqo[q]);
  }

  // ---- scan-kernel tables (scan_kernel.cuh): exact u64 prefixes, no packing ----
  // transient-memory values (peak, peak + act - keep) in units of 2^es bytes: u32 when every
  // value fits, else u64 (es = 0)
  uint32_t es = 16;
  uint64_t emax = 0;
  for (int t = 0; t < T; ++t)
    for (int tp = 0; tp < NT; ++tp)
      for (int b = 0; b < NB; ++b) {
        for (int f : {ACESO_F_ACT, ACESO_F_KEEP, ACESO_F_PEAK})
          if (R(t, tp, b, f) != 0) es = std::min<uint32_t>(es, (uint32_t)__builtin_ctzll((uint64_t)R(t, tp, b, f)));
        emax = std::max(emax, (uint64_t)R(t, tp, b, ACESO_F_PEAK) + R(t, tp, b, ACESO_F_ACT) - R(t, tp, b, ACESO_F_KEEP));
      }
  const bool e64 = (emax >> es) > U32;
  if (e64) es = 0;
  const size_t ew = e64 ? 8 : 4;
  const int nqs = 4 * nch;  // quads incl. the zero-padded tail (4 per chunk)
  std::vector<uint32_t> sqo(nqs, 0u);
  std::vector<std::array<int, 4>> ssig;
  {
    std::map<std::array<int, 4>, int> seen;
    for (int q = 0; q < nqs; ++q) {
      if (4 * q >= L) continue;  // pad quads carry no recompute flags
      std::array<int, 4> key;
      for (int k = 0; k < 4; ++k) key[k] = 4 * q + k < L ? (int)d->op_type[4 * q + k] : -1;
      auto it = seen.find(key);
      if (it == seen.end()) {
        it = seen.emplace(key, (int)ssig.size()).first;
        ssig.push_back(key);
      }
      sqo[q] = (uint32_t)it->second * RUNS * 16u;
    }
  }
  const size_t sc_sx = 0;
  const size_t sc_sk = al(sc_sx + (size_t)RUNS * Lp1 * 32);
  const size_t sc_sd = al(sc_sk + (size_t)RUNS * Lp1 * 16);
  const size_t sc_ss = al(sc_sd + (size_t)NT * ND * Lp1 * 8);
  const size_t sc_sq = al(sc_ss + (size_t)levels * RUNS * L * ew);
  const size_t sc_qo = al(sc_sq + ssig.size() * RUNS * 16 * 32);
  const size_t sc_bytes = al(sc_qo + (size_t)nqs * 4);
  std::vector<unsigned char> sc(sc_bytes, 0);
  {
    auto put64 = [&](size_t off, uint64_t v) { memcpy(&sc[off], &v, 8); };
    auto put32 = [&](size_t off, uint32_t v) { memcpy(&sc[off], &v, 4); };
    auto pute = [&](size_t idx, uint64_t v) {
      if (e64) put64(sc_ss + idx * 8, v);
      else put32(sc_ss + idx * 4, (uint32_t)v);
    };
    auto gete = [&](size_t idx) -> uint64_t {
      if (e64) { uint64_t v; memcpy(&v, &sc[sc_ss + idx * 8], 8); return v; }
      uint32_t v; memcpy(&v, &sc[sc_ss + idx * 4], 4); return v;
    };
    auto Wof = [&](int t, int tp) -> uint64_t {
      return (uint64_t)d->wmem[((int64_t)t * NT + tp) * 2] + (uint64_t)d->wmem[((int64_t)t * NT + tp) * 2 + 1];
    };
    for (int b = 0; b < NB; ++b)
      for (int tp = 0; tp < NT; ++tp) {
        const uint32_t rr = (uint32_t)(b * NT + tp);
        uint64_t PS = 0, PA = 0, PW = 0, PC = 0;
        for (uint32_t j = 0; j <= (uint32_t)L; ++j) {
          const size_t o = (size_t)rr * Lp1 + j;
          put64(sc_sx + o * 32, PS);
          put64(sc_sx + o * 32 + 8, PA);
          put64(sc_sx + o * 32 + 16, PW);
          put64(sc_sx + o * 32 + 24, PC);
          if (j < (uint32_t)L) {
            const int t = d->op_type[j];
            PS += (uint64_t)R(t, tp, b, ACESO_F_FWD_COMP) + R(t, tp, b, ACESO_F_FWD_COMM) +
                  R(t, tp, b, ACESO_F_BWD_COMP) + R(t, tp, b, ACESO_F_BWD_COMM);
            PA += (uint64_t)R(t, tp, b, ACESO_F_ACT);
            PW += Wof(t, tp);
            PC += (uint64_t)R(t, tp, b, ACESO_F_FWD_COMP) + R(t, tp, b, ACESO_F_BWD_COMP);
            put32(sc_sk + o * 16, (uint32_t)R(t, tp, b, ACESO_F_RESHARD));
            put32(sc_sk + o * 16 + 4, (uint32_t)R(t, tp, b, ACESO_F_P2P_BWD));
            pute((size_t)rr * L + j, (uint64_t)R(t, tp, b, ACESO_F_PEAK) >> es);
          }
          if (j > 0) put32(sc_sk + o * 16 + 8, (uint32_t)R(d->op_type[j - 1], tp, b, ACESO_F_P2P_FWD));
        }
        for (int k = 1; k < levels; ++k)
          for (int j = 0; j < L; ++j) {
            const int j2 = std::min(j + (1 << (k - 1)), L - 1);
            const uint64_t v1 = gete(((size_t)(k - 1) * RUNS + rr) * L + j);
            const uint64_t v2 = gete(((size_t)(k - 1) * RUNS + rr) * L + j2);
            pute(((size_t)k * RUNS + rr) * L + j, std::max(v1, v2));
          }
        for (size_t sg = 0; sg < ssig.size(); ++sg)
          for (uint32_t m = 1; m < 16; ++m) {
            uint64_t dS = 0, dA = 0, dC = 0, E1 = 0;
            for (int k = 0; k < 4; ++k) {
              const int t = ssig[sg][k];
              if (t < 0 || !((m >> k) & 1u)) continue;
              dS += (uint64_t)R(t, tp, b, ACESO_F_FWD_COMP) + R(t, tp, b, ACESO_F_FWD_COMM);
              dA += (uint64_t)(R(t, tp, b, ACESO_F_ACT) - R(t, tp, b, ACESO_F_KEEP));
              dC += (uint64_t)R(t, tp, b, ACESO_F_FWD_COMP);
              E1 = std::max(E1, ((uint64_t)R(t, tp, b, ACESO_F_PEAK) + R(t, tp, b, ACESO_F_ACT) -
                                 R(t, tp, b, ACESO_F_KEEP)) >> es);
            }
            const size_t o = sc_sq + (((size_t)sg * RUNS + rr) * 16 + m) * 32;
            put64(o, dS);
            put64(o + 8, dA);
            put64(o + 16, E1);
            put64(o + 24, dC);
          }
      }
    for (int tp = 0; tp < NT; ++tp)
      for (int dp = 0; dp < ND; ++dp) {
        uint64_t acc = 0;
        for (uint32_t j = 0; j <= (uint32_t)L; ++j) {
          put64(sc_sd + (((size_t)tp * ND + dp) * Lp1 + j) * 8, acc);
          if (j < (uint32_t)L) acc += dps_of(d->op_type[j], tp, dp);
        }
      }
    for (int q = 0; q < nqs; ++q) put32(sc_qo + (size_t)q * 4, sqo[q]);
  }

  // ---- device ----
  int ndev = 0;
  if (cudaGetDeviceCount(&ndev) != cudaSuccess || ndev == 0) return fail(ACESO_ENODEV, "no CUDA device");
  if (cuda_device < 0 || cuda_device >= ndev || cuda_device >= 64) return fail(ACESO_EINVAL, "bad device %d", cuda_device);
  int prev_dev = 0;
  CUDA_TRY(cudaGetDevice(&prev_dev));
  CUDA_TRY(cudaSetDevice(cuda_device));
  cudaDeviceProp prop;
  CUDA_TRY(cudaGetDeviceProperties(&prop, cuda_device));
  if (prop.major != 10) {
    cudaSetDevice(prev_dev);
    return fail(ACESO_ENODEV, "device %d is sm_%d%d; libaceso is built for sm_100a", cuda_device, prop.major, prop.minor);
  }
  aceso_ctx *ctx = new aceso_ctx();
  ctx->device = cuda_device;
  ctx->sms = prop.multiProcessorCount;
  ctx->L = L; ctx->T = T; ctx->n_tp = NT; ctx->n_dp = ND; ctx->n_b = NB; ctx->G = d->n_devices;
  ctx->Bg = (uint64_t)d->global_batch;
  ctx->C = (uint64_t)d->mem_capacity;
  ctx->tab = tab;
  ctx->mem_shift = ms;
  ctx->d_blob = nullptr;
  ctx->d_ev = nullptr;
  ctx->packed_ok = packed_ok ? 1 : 0;
  ctx->quad_ok = (quad_ok && packed_ok) ? 1 : 0;
  ctx->d_sc = nullptr;
  ctx->es = es;
  ctx->e64 = e64 ? 1 : 0;
  ctx->qo_words = (uint32_t)nqs;
  ctx->sc_resolve = getenv("ACESO_SCAN_NORESOLVE") ? 0u : 1u;
  ctx->has_alt = d->rec_alt ? 1 : 0;
  ctx->dims_gt = dense_ok ? 0 : 1;
  // default schedule: the event kernel (its packed tables hold the profile), for short models
  // (<= 64 ops) the dense kernel's branch-free per-op accumulation; the scan kernel (exact
  // 64-bit tables) for profiles whose per-op values exceed the packed 32-bit fields
  ctx->kernel = !packed_ok ? 3 : (L <= 64 && dense_ok) ? 2 : 1;
  if (const char *env = getenv("ACESO_KERNEL")) {
    if (!strcmp(env, "quad") && quad_ok && packed_ok) ctx->kernel = 0;
    else if (!strcmp(env, "events") && packed_ok) ctx->kernel = 1;
    else if (!strcmp(env, "dense") && packed_ok) ctx->kernel = 2;  // validated against dense_ok below
    else if (!strcmp(env, "scan")) ctx->kernel = 3;
  }
  ctx->qo_off = (uint32_t)ev_qo;
  ctx->qo_bytes = qo_bytes;
  ctx->has_oct = has_oct ? 1 : 0;
  int rc = ACESO_OK;
  do {
    cudaStream_t st;
    if (cudaStreamCreateWithFlags(&st, cudaStreamNonBlocking) != cudaSuccess) { rc = fail(ACESO_ECUDA, "stream create"); break; }
    cudaError_t e = cudaMalloc(&ctx->d_blob, blob_bytes);
    if (e == cudaSuccess) e = cudaMemcpyAsync(ctx->d_blob, blob.data(), blob_bytes, cudaMemcpyHostToDevice, st);
    if (e == cudaSuccess) e = cudaMalloc(&ctx->d_ev, ev_bytes);
    if (e == cudaSuccess) e = cudaMemcpyAsync(ctx->d_ev, ev.data(), ev_bytes, cudaMemcpyHostToDevice, st);
    if (e == cudaSuccess) e = cudaMalloc(&ctx->d_sc, sc_bytes);
    if (e == cudaSuccess) e = cudaMemcpyAsync(ctx->d_sc, sc.data(), sc_bytes, cudaMemcpyHostToDevice, st);
    if (e == cudaSuccess) e = cudaStreamSynchronize(st);
    cudaStreamDestroy(st);
    if (e != cudaSuccess) { rc = fail(e == cudaErrorMemoryAllocation ? ACESO_ENOMEM : ACESO_ECUDA, "upload: %s", cudaGetErrorString(e)); break; }
    const int nch = (L + 15) / 16;
    // register target: 3 resident CTAs per SM (80 registers) for models of up to 128 chunks;
    // the long models' event kernel runs faster at 2 (measured, 1K-layer GPT: 0.608 vs 0.571 of
    // the HBM roofline at 131,072 candidates, 0.641 vs 0.589 at 1M; GPT-3 1.3B / 13B, T5 and
    // Wide-ResNet lose 11-17% at 2). ACESO_MINB=2|3 overrides.
    ctx->minb = nch > 128 ? 2 : 3;
    ctx->tiles_per_warp = 1;
    if (const char *env = getenv("ACESO_TILES_PER_WARP")) {
      int v = atoi(env);
      if (v >= 1 && v <= 64) ctx->tiles_per_warp = v;
    }
    if (const char *env = getenv("ACESO_MINB")) {
      int v = atoi(env);
      if (v == 2 || v == 3) ctx->minb = v;
    }
    ctx->ev_warps = kWarps;
    ctx->ev_minb = ctx->minb;
    ctx->ev_oct = ctx->has_oct;
    if (const char *env = getenv("ACESO_EV_OCT"))  // measurement knob: 0 = quad lookups
      if (atoi(env) == 0) ctx->ev_oct = 0;
    ctx->ev_sc = (ctx->minb == 2 && ctx->ev_oct) ? 8 : 4;
    if (const char *env = getenv("ACESO_EV_SLOT"))  // measurement knob: 4 or 8 (8 needs 2 CTAs per SM and the octet tables)
      if (atoi(env) == 4 || (atoi(env) == 8 && ctx->minb == 2 && ctx->ev_oct)) ctx->ev_sc = atoi(env);
    {
      const unsigned char *eb = reinterpret_cast<const unsigned char *>(ctx->d_ev);
      ctx->px = reinterpret_cast<const uint4 *>(eb + ev_px);
      ctx->kx = reinterpret_cast<const uint4 *>(eb + ev_kx);
      ctx->pd = reinterpret_cast<const uint64_t *>(eb + ev_pd);
      ctx->st = reinterpret_cast<const uint32_t *>(eb + ev_st);
      ctx->qr = reinterpret_cast<const uint4 *>(eb + ev_qr);
      ctx->qr8 = has_oct ? reinterpret_cast<const uint4 *>(eb + ev_qr8) : nullptr;
      ctx->qo8 = has_oct ? reinterpret_cast<const uint32_t *>(eb + ev_qo8) : nullptr;
      const unsigned char *cb = reinterpret_cast<const unsigned char *>(ctx->d_sc);
      ctx->sx = reinterpret_cast<const uint4 *>(cb + sc_sx);
      ctx->sk = reinterpret_cast<const uint4 *>(cb + sc_sk);
      ctx->sd = reinterpret_cast<const uint64_t *>(cb + sc_sd);
      ctx->ss = reinterpret_cast<const void *>(cb + sc_ss);
      ctx->sq = reinterpret_cast<const uint4 *>(cb + sc_sq);
      ctx->sqo = reinterpret_cast<const uint32_t *>(cb + sc_qo);
    }
    // ACESO_HINT_DENSE: the dense kernel when its tables fit shared memory and the profile fits
    // its packed fields, else the scan kernel
    ctx->dense_kernel = (dense_ok && packed_ok) ? 2 : ctx->quad_ok ? 0 : 3;
    if (ctx->kernel == 2 && !dense_ok) ctx->kernel = packed_ok ? 1 : 3;  // ACESO_KERNEL=dense
    if (const char *env = getenv("ACESO_DENSE_KERNEL"))
      if (!strcmp(env, "quad") && ctx->quad_ok) ctx->dense_kernel = 0;
    for (int kern = 0; kern < 4 && rc == ACESO_OK; ++kern)
      for (uint32_t mode = 1; mode < 8; ++mode) {
        if ((kern == 0 && !ctx->quad_ok) || (kern == 2 && !(dense_ok && packed_ok)) || (kern == 1 && !packed_ok)) {
          ctx->smem[kern][mode] = 0;
          ctx->max_ctas[kern][mode] = 0;
          continue;
        }
        const size_t tabs = ((mode & ACESO_OUT_FULL) ? tab.bytes_full : tab.bytes) + (tab.k_smem ? bytesK : 0u);
        const size_t smem =
            kern == 3   ? (size_t)sc_smem_bytes((uint32_t)(nqs * 4 + 15) & ~15u)
            : kern == 1 ? (size_t)ev_smem_bytes((mode & ACESO_OUT_FULL) != 0, (uint32_t)ctx->ev_warps, ev_sc_for(ctx, mode), qo_bytes)
            : kern == 2 ? ((mode & ACESO_OUT_FULL) ? tab.dbytes_full : tab.dbytes) + kRingBytesPerCta
                        : tabs + kRingBytesPerCta;
        ctx->smem[kern][mode] = smem;
        void *k = kern == 1 ? eval_kernel_for(mode, ctx->ev_minb, 1, 0, ctx->ev_warps, ev_sc_for(ctx, mode), ctx->ev_oct)
                            : eval_kernel_for(mode, ctx->minb, kern, ctx->e64);
        e = cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        int occ = 0;
        if (e == cudaSuccess) e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k, kern == 1 ? 32 * ctx->ev_warps : kThreads, smem);
        if (e != cudaSuccess || occ < 1) {
          rc = fail(ACESO_ECUDA, "kernel setup (kernel %d, mode %u, %zu B smem): %s", kern, mode, smem, cudaGetErrorString(e));
          break;
        }
        ctx->max_ctas[kern][mode] = occ * ctx->sms;
      }
    for (uint32_t mode = 1; mode < 8 && rc == ACESO_OK && ctx->has_alt && packed_ok; ++mode) {
      const size_t smem = (ctx->dims_gt ? 0 : ((mode & ACESO_OUT_FULL) ? tab.dbytes_full : tab.dbytes)) + kRingBytesPerCta;
      void *k = ctx->dims_gt ? dense_dims_kernel_for<true>(mode) : dense_dims_kernel_for<false>(mode);
      e = cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
      int occ = 0;
      if (e == cudaSuccess) e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k, kThreads, smem);
      if (e != cudaSuccess || occ < 1) {
        rc = fail(ACESO_ECUDA, "kernel setup (dimension plane, mode %u, %zu B smem): %s", mode, smem, cudaGetErrorString(e));
        break;
      }
      ctx->dims_smem[mode] = smem;
      ctx->dims_max_ctas[mode] = occ * ctx->sms;
    }
  } while (0);
  cudaSetDevice(prev_dev);
  if (rc != ACESO_OK) {
    if (ctx->d_blob) cudaFree(ctx->d_blob);
    if (ctx->d_ev) cudaFree(ctx->d_ev);
    if (ctx->d_sc) cudaFree(ctx->d_sc);
    delete ctx;
    return rc;
  }
  *out = ctx;
  return ACESO_OK;
}

void aceso_free(aceso_ctx *ctx) {
  if (!ctx) return;
  int prev = 0;
  cudaGetDevice(&prev);
  cudaSetDevice(ctx->device);
  cudaFree(ctx->d_blob);
  cudaFree(ctx->d_ev);
  cudaFree(ctx->d_sc);
  cudaSetDevice(prev);
  delete ctx;
}

size_t aceso_select_buf_bytes(const aceso_ctx *ctx, int64_t n) {
  (void)n;
  if (!ctx) return 0;
  int m = 0;
  for (int kern = 0; kern < 4; ++kern)
    for (int k = 1; k < 8; ++k) m = std::max(m, std::max(ctx->max_ctas[kern][k], ctx->dims_max_ctas[k]));
  m = std::max(m, 4 * ctx->sms);  // per-CTA partials of the eval kernels; select kernel grid
  return (size_t)kSelPartialOff + 16 * (size_t)m;
}

static int eval_impl(aceso_ctx *ctx, const uint8_t *d_codes, const uint64_t *d_hdr, int64_t n,
                     int64_t global_offset, int64_t n_total, uint32_t flags, const aceso_eval_out *out,
                     void *d_sel, unsigned long long *d_global_key, void *stream);

int aceso_eval(aceso_ctx *ctx, const uint8_t *d_codes, const uint64_t *d_hdr, int64_t n,
               int64_t global_offset, int64_t n_total, uint32_t flags, const aceso_eval_out *out,
               void *d_sel, void *stream) {
  return eval_impl(ctx, d_codes, d_hdr, n, global_offset, n_total, flags, out, d_sel, nullptr, stream);
}

int aceso_eval_global(aceso_ctx *ctx, const uint8_t *d_codes, const uint64_t *d_hdr, int64_t n,
                      int64_t global_offset, int64_t n_total, uint32_t flags, const aceso_eval_out *out,
                      void *d_sel, int64_t *d_global_key, void *stream) {
  if (!(flags & ACESO_FUSED_SELECT) || !d_global_key) return fail(ACESO_EINVAL, "aceso_eval_global needs ACESO_FUSED_SELECT and a key address");
  if (((uintptr_t)d_global_key & 7) != 0) return fail(ACESO_EINVAL, "global key not 8-byte aligned");
  return eval_impl(ctx, d_codes, d_hdr, n, global_offset, n_total, flags, out, d_sel,
                   reinterpret_cast<unsigned long long *>(d_global_key), stream);
}

static int eval_impl(aceso_ctx *ctx, const uint8_t *d_codes, const uint64_t *d_hdr, int64_t n,
                     int64_t global_offset, int64_t n_total, uint32_t flags, const aceso_eval_out *out,
                     void *d_sel, unsigned long long *d_global_key, void *stream) {
  if (!ctx) return fail(ACESO_EINVAL, "null context");
  if (n < 0 || global_offset < 0 || n_total < global_offset + n) return fail(ACESO_EINVAL, "bad n / global_offset / n_total");
  if (n_total >= (1ll << 40)) return fail(ACESO_EINVAL, "n_total >= 2^40");
  if (n >= (1ll << 37)) return fail(ACESO_EINVAL, "n >= 2^37");
  const uint32_t mode = flags & 7u;
  if (mode == 0 || (flags & ~(7u | ACESO_HINT_DENSE | ACESO_HINT_OVERLAP | ACESO_PIPE_LITERAL))) return fail(ACESO_EINVAL, "bad flags 0x%x", flags);
  const int kern = (flags & ACESO_HINT_DENSE) ? ctx->dense_kernel : ctx->kernel;
  if (n > 0 && (!d_codes || !d_hdr)) return fail(ACESO_EINVAL, "null codes/headers");
  if ((mode & (ACESO_OUT_SUMMARY | ACESO_OUT_FULL)) && !out) return fail(ACESO_EINVAL, "null outputs");
  if ((mode & ACESO_OUT_SUMMARY) && n > 0 && (!out->iter_ns || !out->max_mem || !out->info)) return fail(ACESO_EINVAL, "null summary array");
  if (mode & ACESO_OUT_FULL) {
    if (out->p_max < ctx->G) return fail(ACESO_EINVAL, "p_max %d < n_devices %d", out->p_max, ctx->G);
    if (n > 0 && (!out->stage_T || !out->stage_mem || !out->stage_comp || !out->stage_comm)) return fail(ACESO_EINVAL, "null stage array");
  }
  if ((mode & ACESO_FUSED_SELECT) && !d_sel) return fail(ACESO_EINVAL, "null select buffer");
  if (((uintptr_t)d_codes & 15) != 0) return fail(ACESO_EINVAL, "codes not 16-byte aligned");
  if (n > 0) {
    PTR_TRY(d_codes, ctx->device);
    PTR_TRY(d_hdr, ctx->device);
    if (mode & ACESO_OUT_SUMMARY) {
      PTR_TRY(out->iter_ns, ctx->device);
      PTR_TRY(out->max_mem, ctx->device);
      PTR_TRY(out->info, ctx->device);
    }
    if (mode & ACESO_OUT_FULL) {
      PTR_TRY(out->stage_T, ctx->device);
      PTR_TRY(out->stage_mem, ctx->device);
      PTR_TRY(out->stage_comp, ctx->device);
      PTR_TRY(out->stage_comm, ctx->device);
    }
  }
  if (mode & ACESO_FUSED_SELECT) PTR_TRY(d_sel, ctx->device);

  EvalParams P = make_params(ctx, n, global_offset, n_total, out, d_sel);
  P.codes = reinterpret_cast<const uint4 *>(d_codes);
  P.hdr = d_hdr;
  P.gkey = d_global_key;
  if (flags & ACESO_PIPE_LITERAL) P.n_minus = 0;

  // tiles per warp: 1 (latency); with ACESO_HINT_OVERLAP on the event kernel, 3 for models of at
  // most 20 chunks (320 ops) and 2 for at most 24 (384 ops), whose per-tile work does not amortise
  // the per-launch prologue and epilogue (measured, 8 streams: GPT-3 1.3B 5.39 / 5.83 / 5.97 G/s
  // with 1 / 2 / 3 tiles; Wide-ResNet 4.66 / 5.04 / 4.99; GPT-3 13B 3.21 / 2.96 / 2.35)
  const int tpw_hint = P.nch <= 20 ? 3 : P.nch <= 24 ? 2 : 1;
  const int tpw = ((kern == 1 || kern == 3) && (flags & ACESO_HINT_OVERLAP) && tpw_hint > 1) ? std::max(tpw_hint, ctx->tiles_per_warp)
                                                                          : ctx->tiles_per_warp;
  const int tiles_per_cta = (kern == 1 ? ctx->ev_warps : kWarps) * tpw;
  const int64_t need = (P.n_tiles + tiles_per_cta - 1) / tiles_per_cta;
  int grid = (int)std::max<int64_t>(1, std::min<int64_t>(need, ctx->max_ctas[kern][mode]));
  if (kern == 3) {
    const int64_t nw = (int64_t)grid * kWarps;
    P.tw_q = (uint32_t)(P.n_tiles / nw);
    P.tw_r = (uint32_t)(P.n_tiles % nw);
    if ((uint64_t)(P.tw_q + 1) * (uint64_t)P.nch >= (1ull << 32) || P.n_tiles >= (1ll << 32))
      return fail(ACESO_EINVAL, "batch too large for one launch (per-warp chunk count >= 2^32)");
  }
  int prev = 0;
  CUDA_TRY(cudaGetDevice(&prev));
  if (prev != ctx->device) CUDA_TRY(cudaSetDevice(ctx->device));
  void *args[] = {&P};
  void *kfn = kern == 1 ? eval_kernel_for(mode, ctx->ev_minb, 1, 0, ctx->ev_warps, ev_sc_for(ctx, mode), ctx->ev_oct)
                        : eval_kernel_for(mode, ctx->minb, kern, ctx->e64);
  cudaError_t e = cudaLaunchKernel(kfn, dim3(grid), dim3(kern == 1 ? 32 * ctx->ev_warps : kThreads), args, ctx->smem[kern][mode],
                                   reinterpret_cast<cudaStream_t>(stream));
  if (prev != ctx->device) cudaSetDevice(prev);
  if (e != cudaSuccess) return fail(ACESO_ECUDA, "eval launch: %s", cudaGetErrorString(e));
  return ACESO_OK;
}

size_t aceso_dims_bytes(int64_t n, int32_t n_ops) {
  if (n < 0 || n_ops < 1) return 0;
  return (size_t)((n + 31) / 32) * (size_t)((n_ops + 15) / 16) * 64;
}

int aceso_pack_dims(const uint8_t *d_rowmajor, int64_t n, int32_t n_ops, uint8_t *d_plane, void *stream) {
  if (n < 0 || n_ops < 1 || n_ops > kMaxOps || (n > 0 && (!d_rowmajor || !d_plane))) return fail(ACESO_EINVAL, "bad argument");
  if (((uintptr_t)d_plane & 1) != 0) return fail(ACESO_EINVAL, "dimension plane not 2-byte aligned");
  PTR_TRY(d_rowmajor, -1);
  PTR_TRY(d_plane, -1);
  if (n == 0) return ACESO_OK;
  const int64_t total = (int64_t)aceso_dims_bytes(n, n_ops) / 2;
  const int grid = (int)std::min<int64_t>((total + 255) / 256, 148 * 16);
  pack_dims_kernel<<<grid, 256, 0, reinterpret_cast<cudaStream_t>(stream)>>>(d_rowmajor, n, n_ops,
                                                                            reinterpret_cast<uint16_t *>(d_plane), total);
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return fail(ACESO_ECUDA, "pack_dims launch: %s", cudaGetErrorString(e));
  return ACESO_OK;
}

int aceso_eval_dims(aceso_ctx *ctx, const uint8_t *d_codes, const uint8_t *d_dims, const uint64_t *d_hdr,
                    int64_t n, int64_t global_offset, int64_t n_total, uint32_t flags,
                    const aceso_eval_out *out, void *d_sel, void *stream) {
  if (!d_dims) return aceso_eval(ctx, d_codes, d_hdr, n, global_offset, n_total, flags, out, d_sel, stream);
  if (!ctx) return fail(ACESO_EINVAL, "null context");
  if (!ctx->has_alt) return fail(ACESO_EINVAL, "dimension plane given but the profile has no rec_alt");
  if (!ctx->packed_ok) return fail(ACESO_ERANGE, "dimension plane: the profile's values exceed the dense kernel's 32-bit fields");
  if (((uintptr_t)d_dims & 1) != 0) return fail(ACESO_EINVAL, "dimension plane not 2-byte aligned");
  if (n < 0 || global_offset < 0 || n_total < global_offset + n) return fail(ACESO_EINVAL, "bad n / global_offset / n_total");
  if (n_total >= (1ll << 40)) return fail(ACESO_EINVAL, "n_total >= 2^40");
  if (n >= (1ll << 37)) return fail(ACESO_EINVAL, "n >= 2^37");
  const uint32_t mode = flags & 7u;
  if (mode == 0 || (flags & ~(7u | ACESO_HINT_DENSE | ACESO_HINT_OVERLAP | ACESO_PIPE_LITERAL))) return fail(ACESO_EINVAL, "bad flags 0x%x", flags);
  if (n > 0 && (!d_codes || !d_hdr)) return fail(ACESO_EINVAL, "null codes/headers");
  if ((mode & (ACESO_OUT_SUMMARY | ACESO_OUT_FULL)) && !out) return fail(ACESO_EINVAL, "null outputs");
  if ((mode & ACESO_OUT_SUMMARY) && n > 0 && (!out->iter_ns || !out->max_mem || !out->info)) return fail(ACESO_EINVAL, "null summary array");
  if (mode & ACESO_OUT_FULL) {
    if (out->p_max < ctx->G) return fail(ACESO_EINVAL, "p_max %d < n_devices %d", out->p_max, ctx->G);
    if (n > 0 && (!out->stage_T || !out->stage_mem || !out->stage_comp || !out->stage_comm)) return fail(ACESO_EINVAL, "null stage array");
  }
  if ((mode & ACESO_FUSED_SELECT) && !d_sel) return fail(ACESO_EINVAL, "null select buffer");
  if (((uintptr_t)d_codes & 15) != 0) return fail(ACESO_EINVAL, "codes not 16-byte aligned");
  if (n > 0) {
    PTR_TRY(d_codes, ctx->device);
    PTR_TRY(d_dims, ctx->device);
    PTR_TRY(d_hdr, ctx->device);
    if (mode & ACESO_OUT_SUMMARY) {
      PTR_TRY(out->iter_ns, ctx->device);
      PTR_TRY(out->max_mem, ctx->device);
      PTR_TRY(out->info, ctx->device);
    }
    if (mode & ACESO_OUT_FULL) {
      PTR_TRY(out->stage_T, ctx->device);
      PTR_TRY(out->stage_mem, ctx->device);
      PTR_TRY(out->stage_comp, ctx->device);
      PTR_TRY(out->stage_comm, ctx->device);
    }
  }
  if (mode & ACESO_FUSED_SELECT) PTR_TRY(d_sel, ctx->device);
  EvalParams P = make_params(ctx, n, global_offset, n_total, out, d_sel);
  P.codes = reinterpret_cast<const uint4 *>(d_codes);
  P.hdr = d_hdr;
  if (flags & ACESO_PIPE_LITERAL) P.n_minus = 0;
  P.dims = d_dims;
  const int64_t need = (P.n_tiles + kWarps - 1) / kWarps;
  const int grid = (int)std::max<int64_t>(1, std::min<int64_t>(need, ctx->dims_max_ctas[mode]));
  int prev = 0;
  CUDA_TRY(cudaGetDevice(&prev));
  if (prev != ctx->device) CUDA_TRY(cudaSetDevice(ctx->device));
  void *args[] = {&P};
  void *k = ctx->dims_gt ? dense_dims_kernel_for<true>(mode) : dense_dims_kernel_for<false>(mode);
  cudaError_t e = cudaLaunchKernel(k, dim3(grid), dim3(kThreads), args, ctx->dims_smem[mode], reinterpret_cast<cudaStream_t>(stream));
  if (prev != ctx->device) cudaSetDevice(prev);
  if (e != cudaSuccess) return fail(ACESO_ECUDA, "eval_dims launch: %s", cudaGetErrorString(e));
  return ACESO_OK;
}

const char *aceso_schedule_name(const aceso_ctx *ctx, uint32_t flags) {
  if (!ctx) return "";
  static const char *const names[4] = {"per-op kernel", "event kernel", "dense kernel", "scan kernel"};
  return names[(flags & ACESO_HINT_DENSE) ? ctx->dense_kernel : ctx->kernel];
}

int aceso_select(aceso_ctx *ctx, const aceso_eval_out *out, int64_t n, int64_t global_offset,
                 int64_t n_total, void *d_sel, void *stream) {
  if (!ctx || !d_sel) return fail(ACESO_EINVAL, "null argument");
  if (n < 0 || global_offset < 0 || n_total < global_offset + n) return fail(ACESO_EINVAL, "bad n / global_offset / n_total");
  if (n > 0 && (!out || !out->iter_ns || !out->max_mem || !out->info)) return fail(ACESO_EINVAL, "null summary");
  if (n > 0) {
    PTR_TRY(out->iter_ns, ctx->device);
    PTR_TRY(out->max_mem, ctx->device);
    PTR_TRY(out->info, ctx->device);
  }
  PTR_TRY(d_sel, ctx->device);
  const int64_t blocks = (n + 255) / 256;
  const int grid = (int)std::max<int64_t>(1, std::min<int64_t>(blocks, 4 * ctx->sms));
  int prev = 0;
  CUDA_TRY(cudaGetDevice(&prev));
  if (prev != ctx->device) CUDA_TRY(cudaSetDevice(ctx->device));
  select_kernel<<<grid, 256, 0, reinterpret_cast<cudaStream_t>(stream)>>>(
      n ? out->iter_ns : nullptr, n ? out->max_mem : nullptr, n ? out->info : nullptr, n, global_offset,
      reinterpret_cast<unsigned char *>(d_sel), n_total, std::max(1u, bitlen((uint64_t)n_total)));
  cudaError_t e = cudaGetLastError();
  if (prev != ctx->device) cudaSetDevice(prev);
  if (e != cudaSuccess) return fail(ACESO_ECUDA, "select launch: %s", cudaGetErrorString(e));
  return ACESO_OK;
}

int aceso_decode_key(int64_t key, int64_t n_total, int *cls, uint64_t *cost, int64_t *index,
                     int *saturated) {
  if (!cls || !cost || !index || !saturated || n_total < 0) return fail(ACESO_EINVAL, "bad argument");
  if (key == INT64_MAX || key < 0) {
    *cls = -1; *cost = 0; *index = -1; *saturated = 0;
    return ACESO_OK;
  }
  const uint32_t ib = std::max(1u, bitlen((uint64_t)n_total));
  const uint64_t k = (uint64_t)key;
  const uint64_t cmax = (1ull << (62 - ib)) - 1;
  *cls = (int)(k >> 62);
  *cost = (k & ((1ull << 62) - 1)) >> ib;
  *index = (int64_t)(k & ((1ull << ib) - 1));
  *saturated = *cost == cmax;
  return ACESO_OK;
}

int aceso_pack_rowmajor(const uint8_t *d_rowmajor, int64_t n, int32_t n_ops, uint8_t *d_tiled,
                        void *stream) {
  if (n < 0 || n_ops < 1 || (n > 0 && (!d_rowmajor || !d_tiled))) return fail(ACESO_EINVAL, "bad argument");
  if (((uintptr_t)d_tiled & 15) != 0) return fail(ACESO_EINVAL, "tiled buffer not 16-byte aligned");
  if (n > 0) {
    PTR_TRY(d_rowmajor, -1);
    PTR_TRY(d_tiled, -1);
  }
  if (n == 0) return ACESO_OK;
  const int64_t total_vec = (int64_t)aceso_tiled_bytes(n, n_ops) / 16;
  const int grid = (int)std::min<int64_t>((total_vec + 255) / 256, 148 * 16);
  pack_kernel<<<grid, 256, 0, reinterpret_cast<cudaStream_t>(stream)>>>(d_rowmajor, n, n_ops, reinterpret_cast<uint4 *>(d_tiled), total_vec);
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return fail(ACESO_ECUDA, "pack launch: %s", cudaGetErrorString(e));
  return ACESO_OK;
}

int aceso_expand(const uint8_t *d_bases, const uint16_t *d_ranks, int32_t n_bases, int32_t n_ops,
                 const aceso_cand *d_cands, int64_t n, uint8_t *d_tiled, uint64_t *d_hdr,
                 void *stream) {
  static_assert(sizeof(aceso_patch) == 8 && sizeof(aceso_cand) == 56, "aceso_cand layout");
  if (n < 0 || n_ops < 1 || n_ops > kMaxOps || n_bases < 1) return fail(ACESO_EINVAL, "bad sizes");
  if (n > 0 && (!d_bases || !d_cands || !d_tiled || !d_hdr)) return fail(ACESO_EINVAL, "null argument");
  if (((uintptr_t)d_tiled & 15) != 0 || ((uintptr_t)d_bases & 15) != 0)
    return fail(ACESO_EINVAL, "bases / tiled output not 16-byte aligned");
  if (n > 0) {
    PTR_TRY(d_bases, -1);
    PTR_TRY(d_ranks, -1);
    PTR_TRY(d_cands, -1);
    PTR_TRY(d_tiled, -1);
    PTR_TRY(d_hdr, -1);
  }
  if (n == 0) return ACESO_OK;
  const int grid = (int)std::max<int64_t>(1, std::min<int64_t>((n + 255) / 256, 148 * 16));
  expand_kernel<<<grid, 256, 0, reinterpret_cast<cudaStream_t>(stream)>>>(
      d_bases, d_ranks, n_bases, n_ops, d_cands, n, reinterpret_cast<uint4 *>(d_tiled), d_hdr);
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return fail(ACESO_ECUDA, "expand launch: %s", cudaGetErrorString(e));
  return ACESO_OK;
}

int64_t aceso_enum_cuts_count(int32_t n_ops, int32_t p) {
  if (n_ops < 1 || n_ops > kMaxOps || p < 1 || p > 8 || p > n_ops) return -1;
  const uint64_t c = binom_sat((uint64_t)n_ops - 1, (uint32_t)p - 1);
  return c >= (1ull << 62) ? -1 : (int64_t)c;
}

int aceso_enum_cuts(int32_t n_ops, int32_t p, uint8_t code, uint64_t hdr, int64_t first, int64_t n,
                    uint8_t *d_tiled, uint64_t *d_hdr, void *stream) {
  const int64_t cnt = aceso_enum_cuts_count(n_ops, p);
  if (cnt < 0) return fail(ACESO_ERANGE, "C(n_ops - 1, p - 1) outside [0, 2^62) or bad n_ops / p");
  if (first < 0 || n < 0 || first + n > cnt) return fail(ACESO_EINVAL, "range [first, first + n) outside [0, %lld)", (long long)cnt);
  if (n > 0 && (!d_tiled || !d_hdr)) return fail(ACESO_EINVAL, "null argument");
  if (((uintptr_t)d_tiled & 15) != 0) return fail(ACESO_EINVAL, "tiled output not 16-byte aligned");
  if (n > 0) {
    PTR_TRY(d_tiled, -1);
    PTR_TRY(d_hdr, -1);
  }
  if (n == 0) return ACESO_OK;
  const int grid = (int)std::max<int64_t>(1, std::min<int64_t>((n + 255) / 256, 148 * 16));
  enum_cuts_kernel<<<grid, 256, 0, reinterpret_cast<cudaStream_t>(stream)>>>(
      n_ops, (uint32_t)(p - 1), code, hdr, first, n, reinterpret_cast<uint4 *>(d_tiled), d_hdr);
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return fail(ACESO_ECUDA, "enumeration launch: %s", cudaGetErrorString(e));
  return ACESO_OK;
}

int aceso_hash(const uint8_t *d_codes, const uint64_t *d_hdr, int64_t n, int32_t n_ops,
               uint64_t *d_hash, void *stream) {
  if (n < 0 || n_ops < 1 || n_ops > kMaxOps || (n > 0 && (!d_codes || !d_hdr || !d_hash)))
    return fail(ACESO_EINVAL, "bad argument");
  if (((uintptr_t)d_codes & 15) != 0) return fail(ACESO_EINVAL, "codes not 16-byte aligned");
  if (n > 0) {
    PTR_TRY(d_codes, -1);
    PTR_TRY(d_hdr, -1);
    PTR_TRY(d_hash, -1);
  }
  if (n == 0) return ACESO_OK;
  const int64_t tiles = (n + 31) / 32;
  const int grid = (int)std::max<int64_t>(1, std::min<int64_t>(tiles, 148 * 32));
  hash_kernel<<<grid, kHashWarps * 32, 0, reinterpret_cast<cudaStream_t>(stream)>>>(
      reinterpret_cast<const uint4 *>(d_codes), d_hdr, n, n_ops, d_hash);
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return fail(ACESO_ECUDA, "hash launch: %s", cudaGetErrorString(e));
  return ACESO_OK;
}

size_t aceso_visited_bytes(int64_t slots) {
  if (slots < 2 || (slots & (slots - 1)) != 0) return 0;
  return (size_t)slots * sizeof(VisitedEntry);
}

int aceso_dedup(const uint64_t *d_hash, int64_t n, uint32_t epoch, void *d_table, int64_t slots,
                uint8_t *d_dup, uint32_t *d_status, void *stream) {
  if (n < 0 || n >= (1ll << 40)) return fail(ACESO_EINVAL, "n outside [0, 2^40)");
  if (epoch < 1 || epoch >= (1u << 23)) return fail(ACESO_EINVAL, "epoch outside [1, 2^23)");
  if (slots < 2 || (slots & (slots - 1)) != 0) return fail(ACESO_EINVAL, "slots must be a power of two >= 2");
  if (!d_table || !d_status || (n > 0 && (!d_hash || !d_dup))) return fail(ACESO_EINVAL, "null argument");
  cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
  CUDA_TRY(cudaMemsetAsync(d_status, 0, sizeof(uint32_t), st));
  PTR_TRY(d_table, -1);
  PTR_TRY(d_status, -1);
  if (n > 0) {
    PTR_TRY(d_hash, -1);
    PTR_TRY(d_dup, -1);
  }
  if (n == 0) return ACESO_OK;
  const int grid = (int)std::max<int64_t>(1, std::min<int64_t>((n + 255) / 256, 148 * 16));
  VisitedEntry *t = reinterpret_cast<VisitedEntry *>(d_table);
  visit_insert_kernel<<<grid, 256, 0, st>>>(d_hash, n, epoch, t, (uint64_t)slots - 1, d_status);
  visit_flag_kernel<<<grid, 256, 0, st>>>(d_hash, n, epoch, t, (uint64_t)slots - 1, d_dup);
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return fail(ACESO_ECUDA, "dedup launch: %s", cudaGetErrorString(e));
  return ACESO_OK;
}

}  // extern "C"
