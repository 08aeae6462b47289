// egemm_internal.h -- declarations shared by the library's translation units (not public).
#pragma once
#include <cstdint>
#include <cuda_runtime.h>
#include "../../include/egemm.h"

namespace egemm {

int num_sms();

// mode 0: round-split (Alg. 1), mode 1: truncate-split (Markidis, NEXT-1 variant),
// mode 2: round-split into bf16 parts (NEXT-3 variant; range_flags not produced)
int launch_split(const float* x, int64_t rows, int64_t cols, int64_t ldx, uint16_t* hi,
                 uint16_t* lo, int64_t ldo, int transpose, uint32_t* range_flags,
                 cudaStream_t stream, int mode = 0, bool pdl = false);
// pdl: launch as the programmatic dependent of the previous kernel in the stream, which must be
// an INDEPENDENT split of the same call (split.cu, PDL hooks); the split then completes only
// after that kernel has.

// Epilogue policies of the tensor-core kernel.
enum EpiKind : int { EPI_STORE = 0, EPI_KNN = 1, EPI_KMEANS = 2 };
// tuning-table op of a GEMM whose B arrives as fp32 (its round-split is part of the call,
// so the table may pick the fused-B kernel); a STORE launch
constexpr int kOpGemmB32 = 3;

// Operands of one launch of the tcgen05 kernel.  hi/lo are fp16 bit patterns, K-major:
// A is rows_a x K (row stride lda elements), B is rows_b x K (row stride ldb).
struct TcOperands {
  const uint16_t* a_hi;
  const uint16_t* a_lo;
  int64_t lda;
  const uint16_t* b_hi;
  const uint16_t* b_lo;
  int64_t ldb;
  // fused A split: fp32 A (rows_a x K, row stride lda_f32); a_hi / a_lo then unused
  const float* a_f32;
  int64_t lda_f32;
  // fused B split: fp32 B stored K x N row-major (row stride ldb_f32); b_hi / b_lo unused
  const float* b_f32;
  int64_t ldb_f32;
};

struct TcConfig {
  int cg;        // 1 or 2 (cta_group)
  int bn;        // MMA N per cluster tile
  int sep;       // separate hh / cross accumulators
  int kc;        // promotion interval in k elements (multiple of 64)
  int terms;     // 3 or 4
  int max_clusters;  // 0 = all SMs
  int fa;        // fused splits allowed, bit mask: 1 = A, 2 = B (in-kernel converter warps)
  int stages;    // smem ring depth (0 = the variant's default)
  int nslices;   // kNN: N-slices per query block (0 = wave-balance formula)
  int nepi;      // kMeans: epilogue warps, 8 or 16 (0 = 16)
  int ares;      // kNN: query tile resident in smem (-1 = when d <= 128, 0 = never)
  int pace;      // STORE: k-pacing (1 = when the workspace has room, 0 = off)
  int fmt;       // operand parts: 0 = fp16 (the paper's round-split), 1 = bf16 (NEXT-3)
  int peel;      // STORE: peel a mostly-empty last wave into a 128 x 128 tail launch (-1 auto, 0 off)
  int ksplit;    // STORE: split-K parts (<= 1: none)
  int tsplit;    // STORE: tail split -- k-parts for the tiles of a last wave at most half full (0 off, 1 on)
};

// Split-K geometry of a STORE launch: k-blocks per part, parts actually used (no empty part),
// rows per part block (the tile height multiple) and the parts buffer's row stride.
struct KSplit {
  int parts, kb_per_part;
  int64_t m_pad, ld;
};
KSplit ksplit_geometry(int64_t M, int64_t N, int64_t K, const TcConfig& cfg);
size_t ksplit_ws_bytes(int64_t M, int64_t N, int64_t K, const TcConfig& cfg);
// Tail split of a STORE launch (cfg.tsplit, no uniform split-K): tiles [u0, u0 + tiles) of the
// unit order -- the last, at most half-full wave of the persistent grid -- run as `parts`
// k-parts of kbpp k-blocks each; parts = 0 when it does not apply.  The workspace holds the
// parts' fp32 sums (parts x tile) per split tile plus a counter per epilogue-warp slab.
struct TailSplit {
  int u0, tiles, parts, kbpp;
  size_t ws_floats, cnt_words;
};
TailSplit tail_geometry(int64_t M, int64_t N, int64_t K, const TcConfig& cfg);
// Workspace bytes of the STORE launch's k-parts: the split-K parts buffer or the tail split's.
size_t parts_ws_bytes(int64_t M, int64_t N, int64_t K, const TcConfig& cfg);

// Environment knobs for experiments, read once per process (tools/; the product path takes
// its configuration from the tuning table and egemm_set_config_ex).
struct Knobs {
  int pace_e, pace_s;  // k-pacing: k-blocks per epoch, slack in epochs (EGEMM_PACE_E / _S)
  int no_pace;         // EGEMM_NO_PACE=1
  int band;            // STORE tile order: m-tiles per band (EGEMM_BAND)
  int a_pf;            // fused A (LDG converters): k-blocks of L2 prefetch (EGEMM_A_PREFETCH)
  int a_staged;        // fused A: TMA-staged in-place conversion when aligned (EGEMM_A_STAGED)
  int as_pf;           // fused A, staged: k-blocks of L2 prefetch (EGEMM_AS_PREFETCH)
  int host_chunk;      // egemm_gemm_host row chunk (EGEMM_HOST_CHUNK, 0 = auto)
  int no_tma_store;    // EGEMM_NO_TMA_STORE=1: STORE epilogue with per-lane row stores (A/B runs)
  int no_pdl;          // EGEMM_NO_PDL=1: no programmatic dependent launches (A/B runs)
  int dbg_no_tma, dbg_no_epi, dbg_mode;  // diagnostics (EGEMM_DEBUG_*; EGEMM_DIAG builds only)
};
const Knobs& knobs();

struct TcEpilogue {
  int kind;
  // EPI_STORE
  float* D;
  int64_t ldd;
  const float* C;
  int64_t ldc;
  uint32_t* sync;      // nullable: 256 B of workspace for the k-pacing counters
  float* partial;      // split-K / tail split: the parts' results, parts_ws_bytes() of workspace
  // EPI_KNN / EPI_KMEANS: per-B-row squared norms (||x_j||^2 or ||c_j||^2)
  const float* bnorm;
  // EPI_KNN
  int knn_k;
  int n_slices;
  float* row_bound;    // [M], bytes 0xFF (NaN = no bound yet) before the launch; nullable
  float* part_key;     // [n_slices][M][knn_k]
  int32_t* part_idx;   // [n_slices][M][knn_k]
  // EPI_KMEANS
  int32_t* assign;     // [M]
  float* best_key;     // [M] ||c_a||^2 - 2 x.c_a
};

int launch_tc(int64_t M, int64_t N, int64_t K, const TcOperands& ops, const TcConfig& cfg,
              const TcEpilogue& epi, cudaStream_t stream);

// apps.cu
int launch_rownorm(const float* x, int64_t rows, int64_t d, int64_t ld, float* out,
                   cudaStream_t stream);
// merge n_lists sorted (key, idx) lists [n_lists][nq][k_in] into the top k per query
int launch_knn_merge(const float* part_key, const int32_t* part_idx, int n_lists, int64_t nq,
                     int k_in, int k, const float* qnorm, int32_t* out_idx, float* out_key,
                     cudaStream_t stream);
size_t kmeans_accumulate_ws(int64_t n, int64_t d, int64_t kc);
int launch_kmeans_accumulate(const float* X, int64_t n, int64_t d, int64_t ldx,
                             const int32_t* assign, const float* best_key, int64_t kc, double* sums,
                             int64_t* counts, double* inertia, void* ws, cudaStream_t stream);
int launch_kmeans_finalize(const double* sums, const int64_t* counts, int64_t kc, int64_t d,
                           float* centroids, cudaStream_t stream);
constexpr int kMaxPeers = 16;
int launch_kmeans_peer_reduce_finalize(const double* const* peer_sums,
                                       const int64_t* const* peer_counts, int nranks, int64_t kc,
                                       int64_t d, double* sums_out, int64_t* counts_out,
                                       float* centroids, cudaStream_t stream);
int launch_fill_c(int64_t M, int64_t N, const float* C, int64_t ldc, float* D, int64_t ldd,
                  cudaStream_t stream);

void set_last_error(const char* fmt, ...);
int read_clock_probe(double* mhz);
int launch_tc_probe(int kind, int N, int K, const void* A, const void* B, const float* C,
                    float* D, cudaStream_t stream);
int read_clock_stats(double* mhz, double* cycles_per_launch, double* launches, int reset);
int read_debug_counter(unsigned long long* value, int reset);
int read_debug_timeline(unsigned long long* out16, int reset);

// tune.cu: the measured configuration table
struct TuneEntry {
  int op = -1;  // EpiKind or kOpGemmB32
  long long m_max = 0, n_max = 0, k_max = 0;
  int cg = 0, bn = 0, sep = 0, kc = 0, fa = 0;
  int terms = 0, stages = 0, nslices = 0, nepi = 0, ares = -1, peel = -1, ksplit = 0, tsplit = -1;
};
bool tune_lookup(int op, long long M, long long N, long long K, TuneEntry* out);
const char* tune_table_path();
int tune_table_size();

}  // namespace egemm
