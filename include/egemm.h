/*
 * egemm.h -- C ABI of the B200-native EGEMM-TC hot path (libegemm.so, sm_100a).
 *
 * Paper: B. Feng et al., "EGEMM-TC: Accelerating Scientific Computing on Tensor Cores with
 * Extended Precision", PPoPP'21.  "P:a-b" = lines of the paper text; "R<n>" =
 * the readings of the paper listed in DESIGN.md.
 *
 * Conventions (all entry points):
 *  - Every pointer argument is a DEVICE pointer owned by the caller, unless stated.
 *  - Calls are asynchronous on `stream` (a cudaStream_t; NULL = legacy default stream), never
 *    synchronise the device, never allocate device memory, and are re-entrant.
 *  - Stream order is kept exactly: the kernels are programmatic dependent launches that may
 *    start their setup (barriers, tensor memory) under the previous kernel's tail, but touch
 *    no global memory before that kernel has completed (griddepcontrol.wait).
 *  - Matrices are row-major with an explicit row stride `ld*` in ELEMENTS.
 *  - fp16 "hi"/"lo" buffers hold IEEE binary16 bit patterns (uint16_t).
 *  - Return value: an egemm_status_t.  Host-side validation is synchronous; EGEMM_ERR_CUDA
 *    reports a launch failure; asynchronous device faults surface at the caller's next sync.
 *    egemm_last_error() gives a thread-local human-readable detail of the last non-OK return.
 *  - There is no CPU fallback: without a usable sm_100a device every compute call returns
 *    EGEMM_ERR_CUDA / EGEMM_ERR_UNSUPPORTED.
 */
#ifndef EGEMM_H
#define EGEMM_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
  EGEMM_OK = 0,
  EGEMM_ERR_INVALID_ARG = 1, /* NULL data, negative size, ld < cols, bad terms / k */
  EGEMM_ERR_UNSUPPORTED = 2, /* alignment / shape outside what the kernels implement */
  EGEMM_ERR_CUDA = 3,        /* a CUDA launch or runtime call failed */
  EGEMM_ERR_WORKSPACE = 4    /* workspace NULL or smaller than the *_workspace_size query */
} egemm_status_t;

/* Static string for a status code. */
const char* egemm_status_string(int status);
/* Thread-local detail message for the last non-OK return of this thread ("" if none). */
const char* egemm_last_error(void);
/* Library version (major*10000 + minor*100 + patch). */
int egemm_version(void);

/*
 * One logical operand matrix, given in fp32 and/or pre-split.
 *  f32   : fp32 values (may be NULL when hi/lo are given and the call does not need fp32).
 *  hi,lo : pre-split fp16 parts from egemm_split, K-MAJOR (rows x K, row stride ld_split);
 *          both NULL = split on the fly into the workspace.
 *  ld    : row stride of f32 in elements.
 *  trans : layout of f32 -- 0: stored as documented for the call; 1: stored transposed.
 *  ld_split: row stride of hi/lo in elements (must be a multiple of 8, i.e. 16-byte rows).
 */
typedef struct {
  const float* f32;
  const uint16_t* hi;
  const uint16_t* lo;
  int64_t ld;
  int trans;
  int64_t ld_split;
} egemm_operand_t;

/*
 * Round-split (Alg. 1 lines 2-3; Fig. 4b):
 *   hi = fp16_RN(x);  lo = fp16_RN(x - (float)hi)
 * RN = round to nearest, ties to even (reading R1).  x - hi is exact in fp32, so hi + lo
 * carries >= 21 mantissa bits for 2^-3 <= |x| < 65520 (Table 1).
 *  x      : rows x cols fp32, row stride ldx (>= cols).
 *  hi, lo : transpose == 0: rows x cols, row stride ldo (>= cols);
 *           transpose == 1: cols x rows (the transpose), row stride ldo (>= rows).
 *  range_flags : nullable device uint32; bits are OR-ed in (never cleared):
 *           bit0 = some |x| >= 65520 or non-finite (hi becomes +-inf / NaN),
 *           bit1 = some 0 < |x| < 2^-3 (below the 21-bit zone; lo loses bits, R4).
 * Out-of-range inputs are not an error (IEEE results), only flagged.
 */
int egemm_split(const float* x, int64_t rows, int64_t cols, int64_t ldx, uint16_t* hi,
                uint16_t* lo, int64_t ldo, int transpose, uint32_t* range_flags, void* stream);

/* Truncate-split, the Markidis variant the paper compares against (Fig. 4a, P:812-824;
 * Table 1 "Markidis 1-5-20"): hi = fp16_RZ(x), lo = fp16_RZ(x - (float)hi).  Same
 * arguments and behaviour as egemm_split.  Feed the result to egemm_gemm as pre-split
 * operands to reproduce the paper's precision comparison (Fig. 7). */
int egemm_split_trunc(const float* x, int64_t rows, int64_t cols, int64_t ldx, uint16_t* hi,
                      uint16_t* lo, int64_t ldo, int transpose, uint32_t* range_flags,
                      void* stream);

/* The bf16 variant of the round-split (the paper's workflow, Sec. 3.1
 * P:596-649, on the bf16 operands of tcgen05 kind::f16): hi = bf16_RN(x), lo = bf16_RN(x - hi),
 * bf16 bit patterns (the top halves of fp32 patterns).  8 + 8 significant bits over the full
 * fp32 exponent range (fp16 parts: 11 + 11 bits within |x| < 65520).  Same arguments as
 * egemm_split without range_flags.  Use with egemm_gemm under operand_format = 1. */
int egemm_split_bf16(const float* x, int64_t rows, int64_t cols, int64_t ldx, uint16_t* hi,
                     uint16_t* lo, int64_t ldo, int transpose, void* stream);

/*
 * Extended-precision GEMM (Alg. 1 "Emulation(D, A, B, C)"):
 *   D[M x N] = A[M x K] * B[K x N] (+ C[M x N] if C != NULL)
 * with A, B round-split into fp16 hi/lo and D accumulated in fp32 on the tensor cores as
 * A_hi B_hi + A_hi B_lo + A_lo B_hi (+ A_lo B_lo when terms == 4) (Alg. 1 l.5-8).
 *  A : f32 trans=0 -> M x K (ld >= K); trans=1 -> K x M (ld >= M).  hi/lo: M x K.
 *  B : f32 trans=0 -> K x N (ld >= N); trans=1 -> N x K (ld >= K).  hi/lo: N x K (K-major).
 *  C : nullable, M x N fp32, row stride ldc.  D: M x N fp32, row stride ldd.  D may not
 *      alias A or B; D may equal C only if ldd == ldc.
 *  terms : 0 (tuning-table default, 3), 3, or 4.
 *  workspace : device scratch of >= egemm_gemm_workspace_size(...) bytes (256-B aligned),
 *      used for the on-the-fly split of operands given only in fp32, for the split-K parts
 *      buffer when the configuration splits K (EGEMM_ERR_WORKSPACE if it does not fit), and,
 *      in its last 256 B, for the k-pacing counters that keep the persistent clusters within a few
 *      k-blocks of each other (L2 reuse of shared tiles).  The pacing is
 *      optional: a workspace that only covers the splits (NULL when both operands are
 *      pre-split) is accepted and the kernel runs unpaced; results are identical.
 * M == 0 or N == 0: no-op.  K == 0: D = C (or 0).
 */
int egemm_gemm(int64_t M, int64_t N, int64_t K, egemm_operand_t A, egemm_operand_t B,
               const float* C, int64_t ldc, float* D, int64_t ldd, int terms, void* workspace,
               size_t workspace_bytes, void* stream);
size_t egemm_gemm_workspace_size(int64_t M, int64_t N, int64_t K, int a_presplit, int b_presplit);

/*
 * The same GEMM on HOST buffers (end-to-end use): D_host[M x N] = A_host[M x K] * B_host[K x N]
 * (row-major, strides lda / ldb / ldd in elements; host memory should be pinned for the
 * copies to be asynchronous).  B is copied and split once; row chunks of A are then copied
 * in, split, multiplied and copied out double-buffered, so both PCIe directions overlap the
 * tensor-core work.  Uses two internal copy streams and events created once per device (the
 * only resources the library creates); concurrent calls on the same device from several
 * host threads are serialised by a per-device lock held while a call enqueues its work and
 * ordered on the device (a call's copies wait for the previous call's last kernel).
 * Asynchronous w.r.t. the host like the other calls: D_host is complete when `stream` has
 * completed.  K must be > 0.
 */
int egemm_gemm_host(int64_t M, int64_t N, int64_t K, const float* A_host, int64_t lda,
                    const float* B_host, int64_t ldb, float* D_host, int64_t ldd, int terms,
                    void* workspace, size_t workspace_bytes, void* stream);
size_t egemm_gemm_host_workspace_size(int64_t M, int64_t N, int64_t K);

/*
 * kNN with the emulated GEMM (the GEMM-based kNN of Garcia et al. [9] with its fp32 GEMM
 * replaced): for each query row q_i of Q[nq x d]
 * the k rows x_j of X[nx x d] with the smallest squared distance
 *   dist_ij = ||q_i||^2 + ||x_j||^2 - 2 q_i . x_j ,
 * ascending by (dist, j), dist clamped to >= 0; self matches are kept (reading R11).
 * Arithmetic (reading R22): q.x_j by Alg. 1 on the tensor core (one promotion
 * chunk over d), then one more tensor-core step adds -||x_j||^2/2 (three exact tf32 parts
 * times ones), key = -2 * that accumulator, dist = max(0, fp32(||q||^2 + key)); the norms
 * are fp32(fp64 sum of squares in ascending t).  Results are bitwise reproducible (the
 * regression model is tests/kernel_model.py).
 *  X     : the references, trans 0.  Either fp32 rows (then split and normed on the fly)
 *          or the "index" from egemm_knn_index: pre-split hi/lo + x_norms (f32 may be NULL).
 *  x_norms : nullable nx fp32 ||x_j||^2 (fp64-accumulated, from egemm_knn_index).
 *  Q     : fp32 query rows (trans 0, ld >= d), split and normed on the fly.
 *  k     : 1 <= k <= 64 and k <= nx (register lists of 16, 32 or 64 entries per thread).
 *  out_idx  : nq x k int32;  out_dist : nq x k fp32.
 */
int egemm_knn(egemm_operand_t X, const float* x_norms, int64_t nx, egemm_operand_t Q, int64_t nq,
              int64_t d, int k, int32_t* out_idx, float* out_dist, void* workspace,
              size_t workspace_bytes, void* stream);
size_t egemm_knn_workspace_size(int64_t nx, int64_t nq, int64_t d, int k, int x_presplit);

/*
 * Merge of sorted partial kNN lists (the second step of the GEMM-based kNN when the
 * references are split -- across the N-slices of one egemm_knn call, or across ranks that
 * each hold a shard of the references): for each query i, the k smallest
 * (key, idx) pairs, ascending, of the union of n_lists lists
 *   keys[l][i][0 .. k_in), idx[l][i][0 .. k_in)   (each list ascending by (key, idx)),
 * with idx < 0 (or INT32_MAX) marking an empty slot.  Indices must be distinct across
 * lists (disjoint reference sets).  out_key[i][t] = key, or max(0, qnorm[i] + key) when
 * qnorm != NULL (the kNN distance, reading R11); empty output slots get idx -1, key +inf.
 *  n_lists in [1, 64], 1 <= k <= k_in * n_lists, k <= 64, k_in <= 1024.  One warp per query;
 *  exact (each pair's rank is counted, no approximation).
 */
int egemm_knn_merge(const float* keys, const int32_t* idx, int n_lists, int64_t nq, int k_in, int k,
                    const float* qnorm, int32_t* out_idx, float* out_key, void* stream);

/* kNN index build: round-split of the references X[nx x d] (row stride ldx) into K-major
 * hi/lo (row stride ld_split, a multiple of 8) and their squared norms ||x_j||^2
 * (fp64-accumulated, rounded once to fp32).  Done once; reused by every egemm_knn call. */
int egemm_knn_index(const float* X, int64_t nx, int64_t d, int64_t ldx, uint16_t* hi, uint16_t* lo,
                    int64_t ld_split, float* norms, void* stream);

/*
 * One Lloyd step of kMeans on the caller's shard of points (the GEMM-based kMeans of [2],
 * P:142-145): assign_i = argmin_j (||c_j||^2 - 2 x_i . c_j) (ties -> lowest j;
 * the key is formed on the tensor core as in egemm_knn, reading R22),
 * then fp64 partial sums sums[j][:] = sum_{a_i = j} x_i (from the fp32 x) and int64 counts.
 * sums / counts / inertia are OVERWRITTEN.  inertia (nullable) = sum_i dist(x_i, c_{a_i}).
 *  X : f32 required (n x d, trans 0); hi/lo optional (pre-split points).
 *  centroids : kc x d fp32 (row stride d).
 */
int egemm_kmeans_step(egemm_operand_t X, int64_t n, int64_t d, const float* centroids, int64_t kc,
                      int32_t* assign, double* sums, int64_t* counts, double* inertia,
                      void* workspace, size_t workspace_bytes, void* stream);
size_t egemm_kmeans_workspace_size(int64_t n, int64_t d, int64_t kc, int x_presplit);

/* After the caller's all_reduce of sums / counts across ranks:
 *   centroids[j] = fp32_RN(sums[j] / counts[j]) for counts[j] > 0; unchanged otherwise (R12). */
int egemm_kmeans_finalize(const double* sums, const int64_t* counts, int64_t kc, int64_t d,
                          float* centroids, void* stream);

/*
 * A launch configuration: the value of one tuning-table entry, and the
 * thread-local override of the table.  0 (or -1 where noted) = "not set / the table's".
 *  cg, bn, sep : tile = cta_group (1, 2), MMA N per tile (128, 224, 256), separate hi*hi
 *                accumulator (0, 1).  Valid: (2,256,0) (2,224,0) (2,128,0|1) (1,128,0|1).
 *  kc          : promotion interval in k (multiple of 64).
 *  stages      : smem ring depth (2..4, per tile what fits 227 KiB; 0 = default).
 *  fused       : -1 table; 0 pre-split operands; 1 fp32 A split inside the GEMM kernel;
 *                2 fp32 B split inside the GEMM kernel (a-2 fused modes).
 *  terms       : 3 or 4 products (0 = the call's / table's).
 *  n_slices    : kNN N-slices per query block (1..16; 0 = table / wave-balance formula).
 *  epi_warps   : kMeans epilogue warps (8 or 16; 0 = table / 16).
 *  a_resident  : kNN query tile resident in smem (-1 = when d <= 128, 0 = never); kMeans
 *                point tile resident (1 = when d <= 128; -1 / 0 = streamed, the default).
 *  pace        : k-pacing of STORE GEMMs (-1 = table / on, 0 = off).
 *  max_clusters: persistent clusters launched (0 = one per SM pair / SM).
 *  operand_format: 0 = fp16 parts (the paper's round-split), 1 = bf16 parts (NEXT-3: the
 *                fp32 exponent range, 8 + 8 bits; egemm_gemm only, pre-split path; pre-split
 *                operands must come from egemm_split_bf16).
 *  tail_peel   : STORE GEMMs with one n-tile of CTA-pair tiles: the rows of a last wave at
 *                most 60 % full run as a second, programmatically dependent launch of
 *                128 x 128 tiles on the SMs the main grid frees (-1 = table, default off;
 *                0 = off, 1 = on).
 *                Same results bit for bit.
 *  ksplit      : STORE split-K (R21's k-parts): K in up to ksplit contiguous parts, each tile's
 *                parts run as separate units, their fp32 results are added in k order (then
 *                + C) by a reduce pass; needs the larger egemm_gemm_workspace_size (0/1 = none).
 *  tail_split  : STORE GEMMs whose persistent grid's last wave is at most half full (also a
 *                single, partly filled wave): only that wave's tiles are cut into 2..4
 *                k-parts (R21) run side by side; each part leaves its fp32 sums in the
 *                workspace and the part that finishes last adds them in k order (+ C) and
 *                stores the tile -- no extra launch.  Uses egemm_gemm_workspace_size's room
 *                (without it the wave runs unsplit) (-1 = table: on for the buckets where it
 *                measured faster -- single-wave K >= 4096 shapes, up to 2x; off for multi-wave
 *                shapes, where it saves SM cycles but not time under the power cap,
 *                profiles/r02_tail_split_ab.json, profiles/r02_tail_split_single_wave.json;
 *                0 = off, 1 = on).  An explicit tile override (cg != 0) starts with both the
 *                tail split and split-K off (the override names one launch configuration).
 */
typedef struct {
  int cg, bn, sep, kc, stages, fused, terms, n_slices, epi_warps, a_resident, pace, max_clusters,
      operand_format, tail_peel, ksplit, tail_split;
} egemm_config_t;

/* Thread-local override of the tuning table for the next calls of this thread: fields set
 * in *cfg replace the table's (a tile override also selects the pre-split path unless
 * `fused` is set).  NULL restores the table.  EGEMM_ERR_UNSUPPORTED for a value the library
 * was not built with. */
int egemm_set_config_ex(const egemm_config_t* cfg);
/* Shorthand: tile (cg, bn, sep) and kc only (fused = 0); all zeros restores the table. */
int egemm_set_config(int cg, int bn, int sep, int kc);
/* The configuration the library would use for op (0 gemm with a pre-split B, 1 knn,
 * 2 kmeans, 3 gemm whose B is fp32, split inside the call) at (M, N, K) = (rows of A /
 * queries / points, columns of B / references / centroids, K / d), after the table and
 * this thread's override. */
int egemm_query_config_ex(int op, int64_t M, int64_t N, int64_t K, egemm_config_t* out);

/* The measured configuration table (replaces the paper's analytic model,
 * Sec. 6): path of the loaded tune_table.json ("" = built-in defaults) and,
 * through *entries (nullable), its number of entries.  Host-only. */
const char* egemm_tune_table(int* entries);
/* The (cg, bn, sep, kc, fused) part of egemm_query_config_ex.  *fused_a (nullable): 1 when
 * an fp32 row-major A would be round-split inside the GEMM kernel, 2 when (op 3) the fp32 B
 * would be, else 0. */
int egemm_query_config(int op, int64_t M, int64_t N, int64_t K, int* cg, int* bn, int* sep,
                       int* kc, int* fused_a);

/* Number of SMs of the current device (0 without a device). */
int egemm_num_sms(void);

/* Debug: effective SM clock (MHz) of CTA 0 over the last tensor-core kernel launch,
 * from clock64 / %globaltimer.  Synchronous (copies a device symbol). */
int egemm_debug_last_clock(double* mhz);

/*
 * Tensor-core precision probe (the profiling workflow of Sec. 3.1, generalised to
 * the floating tcgen05 kinds).  Runs ONE chain of tcgen05.mma (cta_group::1,
 * M = 128) on a single CTA:  D = C + sum over k of A[:, k] * B[:, k]  in the MMA's own
 * arithmetic (fp32 D in TMEM), so D can be compared bitwise with CPU models of the MMA.
 *  kind : 0 = kind::f16 with fp16 operands, 1 = kind::f16 with bf16 operands,
 *         2 = kind::tf32 (fp32 containers; the hardware reads them as tf32).
 *  A    : 128 x K row-major (K contiguous), element = 2 B (kinds 0, 1) or 4 B (kind 2).
 *  B    : N x K row-major (each row one column of the math B), same element type.
 *  C    : nullable 128 x N fp32 addend (NULL = 0, the first MMA overwrites).
 *  D    : 128 x N fp32 output.
 *  N    : multiple of 16 in [16, 256];  K : 1 .. 256 (kinds 0, 1) or 1 .. 128 (kind 2); the
 *         last MMA's missing k are zero.  One MMA consumes 16 (f16/bf16) or 8 (tf32) k.
 * Profiling only (slow, one CTA); the GEMM never calls it.
 */
int egemm_tc_probe(int kind, int N, int K, const void* A, const void* B, const float* C,
                   float* D, void* stream);

/* Debug: running sums of the same probe over every tensor-core launch since the last
 * reset: mean SM clock (MHz), CTA-0 SM cycles per launch (clock-independent kernel cost),
 * number of launches.  reset != 0 zeroes the sums after reading.  Synchronous. */
int egemm_debug_clock_stats(double* mhz, double* cycles_per_launch, double* launches, int reset);

/* Debug: a device event counter bumped by diagnostic kernel modes (a library built with
 * EGEMM_DIAG=1, EGEMM_DEBUG_MODE bit 256: kNN candidate-path entries, one per warp and
 * 32-column group).  reset != 0 zeroes it after reading.  Synchronous. */
int egemm_debug_counter(unsigned long long* value, int reset);

/* Debug: the phase timeline of CTA 0 of the last tensor-core launch (SM clock64 values,
 * 16 slots; written only by a library built with EGEMM_DIAG=1 under EGEMM_DEBUG_MODE bit
 * 2048, else left as they are): [0] entry, [1] setup done (barriers, TMEM, PDL wait),
 * [2] first operand load issued, [3] first MMA issued, [4] last MMA committed, [5] last
 * accumulator chunk received by the epilogue, [6] last result stored, [7] exit barrier
 * passed, [8] first converted stage handed over (fused split), [9] first MMA of the CTA's
 * second unit, [12] last chunk drained, [13] stores' reads done, [14] first TMA issue about to
 * start, [15] producer entered its loop.  out: 16 host words.  reset != 0 zeroes the slots after reading.  Synchronous. */
int egemm_debug_timeline(unsigned long long* out, int reset);

#ifdef __cplusplus
}
#endif
#endif /* EGEMM_H */
