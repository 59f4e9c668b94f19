/*
 * aceso.h — C-ABI of the B200-native batched configuration evaluator for
 * Aceso (Liu et al., "Aceso: Efficient Parallel DNN Training through Iterative
 * Bottleneck Alleviation", EuroSys '24).
 *
 * Citations: "P:Lnn" = line nn of the paper text; "R#" = a reading of
 * an ambiguous passage, listed in DESIGN.md §3 (the register of readings).
 *
 * The library evaluates the paper's performance model (§3.3) over
 * very large batches of candidate parallel configurations (§3.1) and
 * selects the best candidate (Heuristic-1 P:L155, "better" P:L138, Alg. 1/2
 * `Estimate`/`GetBestOf` P:L521-593). Every step runs in the sm_100a kernels of
 * libaceso.so; there is no host or CPU fallback.
 *
 * All profiled costs are integers: times in nanoseconds, sizes in bytes. All
 * accumulation is exact unsigned 64-bit; results are bit-exact and
 * independent of reduction order.
 *
 * Threading: a context may be used from several host threads, on any streams.
 * aceso_last_error() is thread-local.
 */
#ifndef ACESO_H_
#define ACESO_H_

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

/* ------------------------------------------------------------------------- */
/* Status codes (return values).                                             */
/* ------------------------------------------------------------------------- */
#define ACESO_OK       0
#define ACESO_EINVAL  (-1) /* bad argument (null pointer, bad size, bad flags;
                              a device-pointer argument that is plain host memory
                              or another device's memory: every call checks its
                              device pointers with cudaPointerGetAttributes) */
#define ACESO_ERANGE  (-2) /* a profile value does not fit the packed width,
                              keep > act, or a model-wide bound could overflow */
#define ACESO_ECUDA   (-3) /* a CUDA runtime call failed (message in last_error) */
#define ACESO_ENOMEM  (-4) /* device or host allocation failed */
#define ACESO_ENODEV  (-5) /* no usable sm_100 device */

/* ------------------------------------------------------------------------- */
/* Profile: the op-cost database of §3.3.                           */
/* ------------------------------------------------------------------------- */
/* Field order of one profile record rec[type][tpl][b][*] (ns | bytes).       */
enum {
  ACESO_F_FWD_COMP = 0, /* forward compute time of one microbatch (ns)        */
  ACESO_F_FWD_COMM = 1, /* forward tensor-parallel collective time (ns)       */
  ACESO_F_BWD_COMP = 2, /* backward compute time (ns)                         */
  ACESO_F_BWD_COMM = 3, /* backward tensor-parallel collective time (ns)      */
  ACESO_F_ACT      = 4, /* activation bytes kept for backward (no recompute)  */
  ACESO_F_KEEP     = 5, /* bytes kept when the op is recomputed (R3); <= act  */
  ACESO_F_PEAK     = 6, /* transient bytes while the op runs (R4)     */
  ACESO_F_RESHARD  = 7, /* re-partition cost when this op's tp/dp differs from
                           the previous op of the same stage (R13)    */
  ACESO_F_P2P_FWD  = 8, /* send of this op's output to the next stage (R5)    */
  ACESO_F_P2P_BWD  = 9, /* send of this op's input grad to the previous stage */
  ACESO_REC_FIELDS = 10
};

/* Host-side profile description. All pointers are host pointers owned by the
 * caller; aceso_load_profile copies what it needs. Index conventions:
 *   tpl = log2(tensor-parallel degree)   in [0, n_tp)
 *   dpl = log2(data-parallel degree)     in [0, n_dp)
 *   b   = log2(per-GPU microbatch size)  in [0, n_b), b = mbs_log2 - dpl (R8)
 */
typedef struct {
  int32_t n_ops;            /* L: operators in model order, 1..16384          */
  int32_t n_types;          /* T: distinct op types, 1..4096                  */
  int32_t n_tp;             /* tp choices, 1..8                               */
  int32_t n_dp;             /* dp choices, 1..8                               */
  int32_t n_b;              /* per-GPU batch choices, 1..16                   */
  int32_t n_devices;        /* G: simulated devices, 1..255                   */
  const uint16_t *op_type;  /* [n_ops], each < n_types                        */
  const int64_t *rec;       /* [n_types][n_tp][n_b][ACESO_REC_FIELDS]         */
  const int64_t *wmem;      /* [n_types][n_tp][2]: param+grad bytes, optimizer bytes */
  const int64_t *dps;       /* [n_types][n_tp][n_dp]: DP gradient all-reduce ns */
  int64_t mem_capacity;     /* C: device memory in bytes (OOM iff Mem_i > C, R10) */
  int64_t global_batch;     /* Bg: samples per iteration, 1..2^31             */
  const int64_t *rec_alt;   /* nullable; [n_types][n_tp][n_b][ACESO_REC_FIELDS]: the records
                               of each op type under its alternative tensor-parallel
                               partition dimension (§4.2: row- vs column-wise
                               MatMul, input- vs output-channel convolution), same range
                               rules as rec; read for ops a candidate's dimension plane
                               flips (aceso_eval_dims). Parameter bytes and DP sync are
                               those of the default dimension. */
} aceso_profile_desc;

typedef struct aceso_ctx aceso_ctx; /* opaque; owned by the library */

/* Validates and packs the profile, uploads it to `cuda_device` and returns a
 * context. Synchronous. Range rules (ACESO_ERANGE on violation):
 *  - time fields (ns) and dps in [0, 2^32); memory fields (act, keep, peak) and
 *    each wmem entry in [0, 2^40];  keep <= act;
 *  - model-wide: a conservative bound on every iteration time and stage memory
 *    (L * max per-op cost * (Bg + 1)) is < 2^62, so packed keys are exact.
 * Every profile within these rules is evaluated exactly. Schedules: the event,
 * dense and per-op kernels hold per-op values in 32-bit fields (memory in units
 * of 2^m bytes, m = the largest power of two <= 16 dividing every memory value;
 * a recomputed op's time 2(fwd) + bwd < 2^32 ns); a profile outside those
 * fields is served by the scan kernel (exact 64-bit tables) for every call.
 * Returns ACESO_OK and sets *out, or a negative status (see aceso_last_error). */
int aceso_load_profile(const aceso_profile_desc *desc, int cuda_device, aceso_ctx **out);

/* Releases the context and its device memory. Null is ignored. */
void aceso_free(aceso_ctx *ctx);

/* ------------------------------------------------------------------------- */
/* Candidate encoding (configuration representation, §3.1).       */
/* ------------------------------------------------------------------------- */
/* One byte per operator:
 *   bit 0     head : 1 = this op opens a new pipeline stage (stage = contiguous op range)
 *   bits 1..3 tpl  : log2 tensor-parallel degree of this op
 *   bit 4     rc   : 1 = recompute this op in backward
 *   bits 5..7 dpl  : log2 data-parallel degree of this op
 * One 64-bit header per candidate (little-endian bytes):
 *   byte 0 mbs_log2 : log2 of the aggregated microbatch size (R8)
 *   byte 1 p        : number of pipeline stages
 *   bytes 2..7      : reserved, must be 0
 */
#define ACESO_CODE(head, tpl, dpl, rc) \
  ((uint8_t)(((head) & 1) | (((tpl) & 7) << 1) | (((rc) & 1) << 4) | (((dpl) & 7) << 5)))
#define ACESO_HDR(mbs_log2, p) ((uint64_t)((mbs_log2) & 0xff) | ((uint64_t)((p) & 0xff) << 8))

/* Tiled device layout of the op codes: tiles of 32 candidates, chunks of 16 ops.
 * Byte (c, j) of candidate c, op j lives at
 *   ((c / 32) * nch + j / 16) * 512 + (c % 32) * 16 + (j % 16),   nch = ceil(L/16).
 * Pad ops (j >= L) and the pad candidates of a ragged last tile are ignored.
 * A warp's 16-byte loads of one chunk are 512 contiguous bytes. */
#define ACESO_TILE_CANDS 32
#define ACESO_CHUNK_OPS 16

/* Bytes of a tiled buffer holding n candidates of n_ops ops. */
size_t aceso_tiled_bytes(int64_t n, int32_t n_ops);

/* Converts row-major codes [n][n_ops] (device) into the tiled layout (device),
 * writing zero pad bytes. Asynchronous on `stream` (a cudaStream_t; 0 = legacy
 * default stream). */
int aceso_pack_rowmajor(const uint8_t *d_rowmajor, int64_t n, int32_t n_ops,
                        uint8_t *d_tiled, void *stream);

/* ------------------------------------------------------------------------- */
/* Evaluation outputs.                                                        */
/* ------------------------------------------------------------------------- */
/* info word of one candidate */
#define ACESO_INFO_BOTTLENECK(x) ((x) & 0xffu)        /* Heuristic-1 stage   */
#define ACESO_INFO_P(x)          (((x) >> 8) & 0xffu) /* header p                    */
#define ACESO_INFO_OOM           (1u << 16)           /* some stage has Mem_i > C    */
#define ACESO_INFO_INVALID       (1u << 17)           /* not a configuration         */
#define ACESO_INFO_REASONS(x)    ((x) >> 18)          /* mask of ACESO_R_* below     */

/* Invalid-configuration reasons (bitmask; every violated rule is reported). */
#define ACESO_R_HEAD0   (1u << 0) /* op 0 does not open a stage                         */
#define ACESO_R_NSTAGE  (1u << 1) /* number of heads != p                               */
#define ACESO_R_PRANGE  (1u << 2) /* p == 0 or p > G                                    */
#define ACESO_R_GSTAGE  (1u << 3) /* tp*dp differs between two ops of one stage */
#define ACESO_R_GSUM    (1u << 4) /* sum over stages of tp*dp != G (R9)                 */
#define ACESO_R_DPMBS   (1u << 5) /* dp > mbs for some op (per-GPU batch < 1)   */
#define ACESO_R_TABLE   (1u << 6) /* tpl >= n_tp, dpl >= n_dp or b >= n_b               */
#define ACESO_R_MBS     (1u << 7) /* mbs > Bg or Bg % mbs != 0                          */
#define ACESO_R_HDR     (1u << 8) /* reserved header bytes not zero                     */

/* Device output arrays (SoA). Pointers are device pointers owned by the caller.
 * Summary (ACESO_OUT_SUMMARY):
 *   iter_ns[n]  iteration time  max_i T_i (Eq. 2, R1)          0 if invalid
 *   max_mem[n]  max_i Mem_i (Eq. 1 + P:L232 + P:L234)          0 if invalid
 *   info[n]     bottleneck | p<<8 | status | reasons<<18
 * Full (ACESO_OUT_FULL), stage-major [p_max][n], written for valid candidates
 * and stages i < p only (other entries untouched):
 *   stage_T    T_i = sum_k S_k + (N-1) S_i + D_i
 *   stage_mem  Mem_i = Wst_i + min(p-i, N) A_i + E_i
 *   stage_comp N * sum_j (fwd_comp + bwd_comp + rc*fwd_comp)
 *   stage_comm N * sum_j (fwd_comm + bwd_comm + rc*fwd_comm + rs_j) + N*p2p_i + D_i
 */
typedef struct {
  uint64_t *iter_ns;
  uint64_t *max_mem;
  uint32_t *info;
  uint64_t *stage_T;
  uint64_t *stage_mem;
  uint64_t *stage_comp;
  uint64_t *stage_comm;
  int32_t p_max; /* row count of the stage arrays; must be >= n_devices for FULL */
} aceso_eval_out;

#define ACESO_OUT_SUMMARY  1u /* write iter_ns, max_mem, info                   */
#define ACESO_OUT_FULL     2u /* also write the per-stage arrays                 */
#define ACESO_FUSED_SELECT 4u /* reduce the batch argmin into d_sel (fused K2)   */
#define ACESO_HINT_DENSE   8u /* schedule hint: candidates change tp/dp or
                                 recompute at most ops (e.g. uniformly random
                                 encodings); selects the per-op kernel instead
                                 of the event kernel. Results are identical.  */
#define ACESO_HINT_OVERLAP 16u /* schedule hint: the caller keeps several
                                 independent batches in flight on different
                                 streams; for models of at most 384 ops the event
                                 kernel then launches a half or a third of the
                                 CTAs and each warp walks two tiles (at most 384
                                 ops) or three (at most 320) (per-launch prologue/
                                 epilogue amortised; higher throughput, longer
                                 single-launch latency); longer models are
                                 unaffected.
                                 Results are identical.                         */

#define ACESO_PIPE_LITERAL 32u /* Eq. 2 as printed: the steady phase runs N
                                 microbatches of stage i, T_i = sum_k S_k + N S_i + D_i;
                                 default (reading R1): N - 1, the 1F1B
                                 makespan on uniform stages. Applies to every output. */

/* ------------------------------------------------------------------------- */
/* Selection (Alg. 1 GetBestOf P:L543, Alg. 2 `perf < init_perf` P:L576).     */
/* ------------------------------------------------------------------------- */
/* Order: lexicographic on (class, cost, global index); class 0 = feasible
 * (cost = iteration time), class 1 = out of memory (cost = max_i Mem_i, R12);
 * invalid candidates are excluded. Result written to the first 32 bytes of the
 * caller's select buffer:                                                   */
typedef struct {
  int64_t key;       /* packed key for an all-reduce MIN across ranks:
                        class<<62 | min(cost, 2^(62-IB)-1)<<IB | index,
                        IB = bit length of n_total; INT64_MAX if nothing valid */
  uint64_t cls_cost; /* exact class<<62 | cost; UINT64_MAX if nothing valid    */
  int64_t index;     /* exact global index of the winner; -1 if nothing valid  */
  uint64_t reserved;
} aceso_select_result;

/* Size in bytes of the select buffer for a batch of n candidates (result +
 * per-CTA partials + a completion counter). The buffer must be zero-filled once
 * at allocation; every call leaves it reusable. One buffer per in-flight call. */
size_t aceso_select_buf_bytes(const aceso_ctx *ctx, int64_t n);

/* Evaluates candidates [0, n) of a batch whose first candidate has global index
 * `global_offset` in a job of `n_total` candidates (sharding, §8e).
 *   d_codes : tiled op codes (device)        d_hdr : [n] headers (device)
 *   flags   : OR of ACESO_OUT_SUMMARY / ACESO_OUT_FULL / ACESO_FUSED_SELECT, plus
 *             optionally ACESO_HINT_DENSE / ACESO_HINT_OVERLAP. Schedules (results
 *             are bit-identical):
 *             the event kernel (default for n_ops > 64) walks each candidate's
 *             stage heads and tp/dp changes and takes run sums from position-prefix
 *             tables; the dense kernel (default for n_ops <= 64, and with
 *             ACESO_HINT_DENSE) accumulates every op branch-free under its own record;
 *             the per-op kernel accumulates every op with quad-signature sums; the
 *             scan kernel streams each warp's tiles as one contiguous range and walks
 *             the dirty chunks (heads, tp/dp changes, recompute flags) with exact
 *             64-bit prefix tables (the schedule for profiles outside the packed
 *             fields, see aceso_load_profile). The dense and per-op kernels stage
 *             their tables in shared memory, so for profiles whose tables exceed
 *             ~200 KB the event (or scan) kernel serves the hint too. Environment
 *             variables read by aceso_load_profile (measurement and test knobs;
 *             results never change): ACESO_KERNEL=quad|events|dense|scan (default
 *             schedule), ACESO_DENSE_KERNEL=quad (schedule of the dense hint),
 *             ACESO_MINB=2|3 (register target: resident CTAs per SM),
 *             ACESO_EV_SLOT=4|8 (event kernel: chunks per ring slot; 8 only at 2
 *             CTAs per SM), ACESO_TILES_PER_WARP=k (event / scan kernel: tiles per
 *             warp per launch), ACESO_SCAN_NORESOLVE=1 (scan kernel: recompute-only
 *             chunks resolved in the per-lane walk).
 *   out     : host struct of device pointers (may be null if no OUT_* flag)
 *   d_sel   : select buffer (device), required with ACESO_FUSED_SELECT
 *   stream  : cudaStream_t
 * Asynchronous; no allocation, no host synchronisation. n == 0 is valid (the
 * select result becomes "nothing valid"). ACESO_EINVAL if n >= 2^37 or
 * n_total >= 2^40 (far beyond device memory at one byte per op). */
int aceso_eval(aceso_ctx *ctx, const uint8_t *d_codes, const uint64_t *d_hdr, int64_t n,
               int64_t global_offset, int64_t n_total, uint32_t flags,
               const aceso_eval_out *out, void *d_sel, void *stream);

/* Name of the kernel aceso_eval runs for `flags` on this context ("event kernel",
 * "dense kernel", "per-op kernel" or "scan kernel"; "" for a null context). Static
 * string, owned by the library. Host only. */
const char *aceso_schedule_name(const aceso_ctx *ctx, uint32_t flags);

/* ------------------------------------------------------------------------- */
/* Tensor-parallel partition dimension per operator (§4.2 fine-tuning,        */
/* P:L263-265).                                                               */
/* ------------------------------------------------------------------------- */
/* Dimension plane: one bit per op (1 = the op runs under its alternative
 * partition dimension and reads rec_alt), tiled like the codes: the 16 bits of
 * chunk k of candidate c are the little-endian u16 at
 *   ((c / 32) * nch + k) * 64 + (c % 32) * 2,   bit (j % 16) = op j = 16 k + j % 16.
 * Bits of pad ops (j >= n_ops) are ignored. */
size_t aceso_dims_bytes(int64_t n, int32_t n_ops);

/* Row-major dimension bytes [n][n_ops] (device, nonzero = alternative) -> the tiled
 * plane (device, 2-byte aligned; pad bits zero). Async on `stream`. */
int aceso_pack_dims(const uint8_t *d_rowmajor, int64_t n, int32_t n_ops, uint8_t *d_plane, void *stream);

/* aceso_eval with a dimension plane (nullable: identical to aceso_eval). Every op
 * whose bit is set uses the alternative-dimension records in every term of the
 * model (its compute, collectives, memory, reshard and p2p). Same flags, outputs,
 * selection and errors as aceso_eval, plus: ACESO_EINVAL if the context has no
 * rec_alt or d_dims is not 2-byte aligned; ACESO_ERANGE if the profile's values
 * exceed the 32-bit packed fields (see aceso_load_profile). Schedule: the dense
 * kernel (per-op accumulation, records read per op under type or type + T), its
 * tables in shared memory when they fit, else in global memory. */
int aceso_eval_dims(aceso_ctx *ctx, const uint8_t *d_codes, const uint8_t *d_dims, const uint64_t *d_hdr,
                    int64_t n, int64_t global_offset, int64_t n_total, uint32_t flags,
                    const aceso_eval_out *out, void *d_sel, void *stream);

/* aceso_eval with the global selection fused into the launch (§8e, NVSwitch-native
 * variant): flags must include ACESO_FUSED_SELECT; after writing the batch's select
 * result, the grid's last CTA also applies atomicMin_system of the packed key to
 * *d_global_key — a device address on this GPU or an NVLink peer-mapped address of
 * another GPU's memory (e.g. the rank-0 buffer of a symmetric-memory allocation), so
 * every rank's launch joins one job-wide key without a separate collective. The
 * caller initialises the key to INT64_MAX and reads it after all ranks' launches
 * complete; decode it with aceso_decode_key (a saturated key needs the exact
 * pairs of the select buffers, as with the NCCL path). 8-byte aligned. */
int aceso_eval_global(aceso_ctx *ctx, const uint8_t *d_codes, const uint64_t *d_hdr, int64_t n,
                      int64_t global_offset, int64_t n_total, uint32_t flags, const aceso_eval_out *out,
                      void *d_sel, int64_t *d_global_key, void *stream);

/* Argmin over an already written summary (iter_ns, max_mem, info) of n
 * candidates; same order and result layout as the fused select. Async. */
int aceso_select(aceso_ctx *ctx, const aceso_eval_out *out, int64_t n, int64_t global_offset,
                 int64_t n_total, void *d_sel, void *stream);

/* Decodes a packed key. *saturated = 1 when the cost field is clamped (the
 * exact cls_cost must then be used). Returns ACESO_OK; for INT64_MAX sets
 * *cls = -1, *index = -1. */
int aceso_decode_key(int64_t key, int64_t n_total, int *cls, uint64_t *cost, int64_t *index,
                     int *saturated);

/* ------------------------------------------------------------------------- */
/* On-device candidate generation (Table 1): */
/* a candidate is a base configuration plus up to 6 byte-range patches, the   */
/* form every reconfiguration primitive of the search driver takes; the      */
/* kernel writes the expanded candidates directly in the tiled layout.       */
/* ------------------------------------------------------------------------- */
enum {
  ACESO_PATCH_NONE = 0,
  ACESO_PATCH_MASK = 1,    /* ops [a, b): c = (c & v0) | v1                          */
  ACESO_PATCH_ADD = 2,     /* ops [a, b): tp field += (int8)v0, dp field += (int8)v1;
                              the caller keeps every field inside [0, 7]           */
  ACESO_PATCH_RANK_RC = 3  /* ops j in [a, b) with rank[v2 & 1][j] < (v0 | v1 << 8):
                              recompute bit set (v2 bit 1 = 0) or cleared (= 1)      */
};
typedef struct {
  uint16_t a, b;     /* op range [a, b), b <= n_ops                                */
  uint8_t kind;      /* ACESO_PATCH_*                                             */
  uint8_t v0, v1, v2;
} aceso_patch;       /* 8 bytes                                                    */
typedef struct {
  uint32_t base;     /* row of the bases array                                    */
  uint8_t mbs_log2;  /* header byte 0 of the candidate                            */
  uint8_t p;         /* header byte 1 (stage count)                               */
  uint8_t n_patch;   /* patches applied in order, <= 6                             */
  uint8_t reserved;
  aceso_patch patch[6];
} aceso_cand;        /* 56 bytes                                                   */

/* Expands n candidates.
 *   d_bases : [n_bases][stride] u8 row-major base encodings, stride = 16 *
 *             ceil(n_ops / 16), bytes >= n_ops zero (device)
 *   d_ranks : [n_bases][2][stride] u16 ranks for ACESO_PATCH_RANK_RC (device; may
 *             be null when no candidate uses that patch)
 *   d_cands : [n] aceso_cand (device)
 *   d_tiled : tiled output, aceso_tiled_bytes(n, n_ops) bytes (device, 16-byte
 *             aligned); d_hdr : [n] u64 headers out (mbs_log2 | p << 8)
 * Out-of-range base indices or patch ranges are clamped away (no access outside
 * the arrays); the result is then unspecified. Async on `stream`. */
int aceso_expand(const uint8_t *d_bases, const uint16_t *d_ranks, int32_t n_bases, int32_t n_ops,
                 const aceso_cand *d_cands, int64_t n, uint8_t *d_tiled, uint64_t *d_hdr,
                 void *stream);

/* ------------------------------------------------------------------------- */
/* Exhaustive stage-partition enumeration (the Exp#4     */
/* mathematical-programming baseline explores a pruned configuration space    */
/* with the same performance model).                               */
/* ------------------------------------------------------------------------- */
/* Number of candidates of a family: C(n_ops - 1, p - 1) (the (p-1)-subsets of the
 * cut positions 1 .. n_ops-1). -1 if 1 <= p <= min(8, n_ops) does not hold or the
 * count is >= 2^62. Host only, no device access. */
int64_t aceso_enum_cuts_count(int32_t n_ops, int32_t p);
/* Writes candidates [first, first + n) of the family (p, code, hdr) in the tiled
 * layout: candidate r has stage heads at op 0 and at the cuts of the r-th
 * (p-1)-subset of {1, ..., n_ops-1} in colex order (r = sum_i C(cut_i - 1, i),
 * cuts ascending, i = 1..p-1); every op carries `code` with its head bit cleared
 * (tp, dp and recompute bits: a stage-uniform configuration); headers = hdr.
 *   d_tiled : aceso_tiled_bytes(n, n_ops) bytes (device, 16-byte aligned)
 *   d_hdr   : [n] u64 (device)
 * ACESO_ERANGE for a bad family, ACESO_EINVAL for a range outside the family.
 * Async on `stream`. */
int aceso_enum_cuts(int32_t n_ops, int32_t p, uint8_t code, uint64_t hdr, int64_t first, int64_t n,
                    uint8_t *d_tiled, uint64_t *d_hdr, void *stream);

/* ------------------------------------------------------------------------- */
/* Configuration dedup ("skip configurations     */
/* already explored"). The encoding above is canonical (one byte per op plus   */
/* the header), so equal configurations have equal bytes and hash equal.       */
/* ------------------------------------------------------------------------- */
/* 64-bit hash of every candidate: the row-major byte string (L code bytes, then
 * the 8 header bytes little-endian, zero-padded to a multiple of 8) read as
 * little-endian u64 words w_0..w_{m-1}; with mix(x) = splitmix64's finalizer
 *   (x ^= x >> 30; x *= 0xBF58476D1CE4E5B9; x ^= x >> 27; x *= 0x94D049BB133111EB;
 *    x ^= x >> 31),
 *   h = mix(0x243F6A8885A308D3 + sum_i mix(w_i ^ (i + 1) * 0x9E3779B97F4A7C15))  (mod 2^64),
 *   h = 1 if h == 0 (0 marks an empty visited-set slot). Words mix independently
 *   (position-tagged), so the kernel streams them with full instruction parallelism.
 *   d_codes : tiled codes (device, 16-byte aligned)   d_hdr : [n] headers
 *   d_hash  : [n] u64 output (device). Async on `stream`. */
int aceso_hash(const uint8_t *d_codes, const uint64_t *d_hdr, int64_t n, int32_t n_ops,
               uint64_t *d_hash, void *stream);

/* Visited set: open addressing over `slots` (a power of two >= 2) entries of 16
 * bytes {hash, tag} in caller-owned device memory, zero-filled once. A call with
 * epoch e (1 <= e < 2^23, increasing across calls) inserts the n hashes and
 * writes d_dup[i] = 1 if hash i was inserted by an earlier call or by a lower
 * index of this call, else 0 (deterministic first occurrence). A full table is
 * reported asynchronously: *d_status = 1 (device u32, zeroed by the call) and
 * d_dup is unspecified. Entries: {hash, ~(epoch << 40 | index) max-reduced}.
 * Two launches on `stream` (insert, then flag). n < 2^40. */
size_t aceso_visited_bytes(int64_t slots);
int aceso_dedup(const uint64_t *d_hash, int64_t n, uint32_t epoch, void *d_table, int64_t slots,
                uint8_t *d_dup, uint32_t *d_status, void *stream);

/* Message of the last failing call on this thread ("" if none). */
const char *aceso_last_error(void);

/* Library version string. */
const char *aceso_version(void);

#ifdef __cplusplus
}
#endif
#endif /* ACESO_H_ */
