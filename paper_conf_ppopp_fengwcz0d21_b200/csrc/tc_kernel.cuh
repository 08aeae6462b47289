// tc_kernel.cuh -- the EGEMM tensor-core kernel for sm_100a (tcgen05 + TMA + TMEM), included
// by the translation units that instantiate its variants (tc_store.cu, tc_fused.cu,
// tc_knn.cu, tc_kmeans.cu; split for parallel compilation) and by gemm_tc.cu (host side).
//
// Computes, per output element, the emulated extended-precision product of Alg. 1
// (PAPER.md P:739-757):  sum_k  A_hi*B_hi + A_hi*B_lo + A_lo*B_hi (+ A_lo*B_lo if terms=4)
// on fp16 tensor cores with fp32 accumulation (Alg. 1 l.5-8; "data combination through the
// fp32 accumulator"), and hands the fp32 result to an epilogue policy:
//   EPI_STORE   D = result (+ C)                          (Alg. 1's D = A x B + C)
//   EPI_KNN     key = ||x_j||^2 - 2 q.x_j, register top-k  (kNN case study)
//   EPI_KMEANS  key = ||c_j||^2 - 2 x.c_j, running argmin (kMeans case study)
//
// B200 design:
//  * warp-specialised persistent kernel, 12 warps: w0 TMA producer, w1 MMA issuer (one
//    elected lane; leader CTA only when CG == 2), w2 TMEM allocator, w3 norm warp (kNN /
//    kMeans) or idle, w4..w11 epilogue (two warps per TMEM lane quarter, each owning BN/2
//    columns).
//  * kNN / kMeans ("norm MMA", reading R22 in DESIGN.md): after a tile's last product MMA one
//    more tcgen05.mma kind::tf32 adds y_j = -||b_j||^2 / 2 to every row of column j (A' = rows
//    of ones, B' = the three tf32 parts of y_j written into the stage by the norm warp), so
//    the accumulator holds a.b_j - ||b_j||^2/2 = -key/2: the tensor core broadcasts the norms
//    and the epilogue only compares accumulators (no per-thread norm loads, no FMA).
//  * operands: pre-split fp16 hi/lo, K-major, loaded by TMA into 128-B-swizzled stages
//    (BK = 64 fp16 = one swizzle atom row) in a STAGES-deep full/empty mbarrier ring.
//  * CG == 2: cta_group::2 pair, UMMA M = 256, each CTA stages its 128 A rows and BN/2 B
//    rows; the leader issues the MMAs, commits multicast to both CTAs.
//  * accumulation: two TMEM accumulator buffers used in ping-pong per k-chunk of Kc
//    elements ("promotion"): the MMA warp fills one while the epilogue warps drain the
//    other into an fp32 register running total with round-to-nearest adds.  This bounds
//    the error of the tensor core's internal fp32 accumulation (P:729-737 report only 21
//    matching bits) to Kc-long sums -- the TMEM analogue of the paper's FRAG caching of
//    C across the k-loop (Table 2).  SEP additionally keeps the
//    hi*hi and cross products in separate accumulators (needs 4 x BN TMEM columns).
//  * tiles: BN = 256, 224 (whole waves of 74 clusters for N = 8192 at short M) or 128 per
//    CTA pair; CG == 1: 128 x 128.
//  * fused splits (a converter warpgroup in front, setmaxnreg 96 / 56 / 176): FA converts
//    fp32 A (LDG, or AS: the TMA-staged fp32 tile converted in place in the stage's A
//    region); FB converts TMA-staged fp32 B (K x N row-major) into the K-major B stage.
//  * kNN epilogue (KREG): the tile is loaded from TMEM and released before ranking; the two
//    column groups of a row filter on the union of their lists (smem exchange per tile) and
//    the row's N-slices share that bound through global memory.
#pragma once
#include <cuda.h>
#include <cudaTypedefs.h>
#include <cuda_runtime.h>
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <atomic>
#include <mutex>
#include "egemm_internal.h"
#include "ptx.cuh"

namespace egemm {


__device__ __forceinline__ unsigned long long globaltimer_ns() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}

// Diagnostic kernel modes (EGEMM_DEBUG_* environment, tools/diag_*.py) exist only in a
// library built with -DEGEMM_DIAG=1 (build.py defines=["EGEMM_DIAG=1"]); in the product
// build every diagnostic branch below is a compile-time false and disappears.
#ifndef EGEMM_DIAG
#define EGEMM_DIAG 0
#endif
constexpr bool kDiag = EGEMM_DIAG != 0;
#define DIAG_NO_TMA (kDiag && p.debug_no_tma)
#define DIAG_NO_EPI (kDiag && p.debug_no_epi)
#define DIAG_MODE(bits) (kDiag && (p.debug_mode & (bits)))
// phase timeline of CTA 0 (EGEMM_DEBUG_MODE bit 2048; egemm_debug_timeline): slot i <- clock64
#define TL(i) do { if (DIAG_MODE(2048) && blockIdx.x == 0) p.probe[8 + (i)] = clock64(); } while (0)

constexpr int kBM = 128;       // rows per CTA (TMEM lanes)
constexpr int kBK = 64;        // k elements per stage (128 B of fp16: one SW128 row)
constexpr int kKnnMerge = 8;   // kNN: list entries handed over per merge round (8 KiB scratch)

struct KParams {
  int M, N;
  int num_kb;       // ceil(K / 64)
  int kb_per_chunk; // Kc / 64
  int ksplit;       // STORE: k-parts per tile (1 = none); part results go to D's row block ks
  int kb_per_part;  // k-blocks per part
  int m_pad;        // rows per part block of D (a multiple of the tile height)
  int terms;
  int m_tiles, n_tiles;
  int num_units;
  int n_slices, tiles_per_slice;  // EPI_KNN
  // epilogue
  float* D;
  int64_t ldd;
  const float* C;
  int64_t ldc;
  int vec_ok;
  const float* bnorm;
  int knn_k;
  float* row_bound;  // kNN (nullable): per query row, a shared upper bound on its k-th key
  float* part_key;
  int32_t* part_idx;
  int32_t* assign;
  float* best_key;
  // fused A split (FA): fp32 A, row stride lda_f32; vec_a = 16-B aligned rows
  const float* a_f32;
  int64_t lda_f32;
  int vec_a;
  int a_pf;         // FA: k-blocks of fp32 A prefetched into L2 ahead of its loads (0: off)
  int a_staged;     // FA: tm_ahi maps fp32 A with 32-column 128-B-swizzled boxes (AS variant)
  int K;
  int debug_no_tma;  // EGEMM_DEBUG_NO_TMA=1: skip operand loads (timing diagnostics only)
  int debug_no_epi;  // EGEMM_DEBUG_NO_EPI=1: skip the promotion's TMEM reads (diagnostics)
  uint32_t* sync;    // nullable: kSyncR epoch counters (zeroed per launch) for the k-pacing
  int pace_e, pace_s;  // k-blocks per epoch, slack in epochs
  int band_m;          // STORE tile order: m-tiles per band
  int fb;            // fused B split (host-side dispatch flag; tm_bhi maps the fp32 B)
  int bf16;          // operands are bf16 hi / lo parts (NEXT-3 variant), not fp16
  int pdl_wait;      // a peeled tail launch (programmatic dependent launch of the main grid)
  int tma_store;     // STORE: D through TMA stores (tm_d; no C, aligned D); else per-lane stores
  unsigned long long* probe;  // device clock probe: [0..3] last launch, [4..6] running sums, [7] counter
  int debug_mode;    // EGEMM_DEBUG_MODE bits (diagnostics): 1 extra commit per k-block;
                     // 2048 phase timeline of CTA 0; 4096 staged fused-A converters skip the
                     // conversion (wrong results; bounds its cost);
                     // with NO_TMA: 2 MMA warp ignores the full barriers (producer idle),
                     // 4 no per-k-block commits; 1024 (fused-A / resident-A variants) no B
                     // loads after the ring's first fill
  // STORE tail split (R21's k-parts for the last, partly filled wave only): units >= tail_u0
  // are k-parts (tail_parts per tile, tail_kbpp k-blocks each) of the tiles tail_u0, ...;
  // each part leaves its fp32 sum in fix_ws and the last part to finish a warp's slab (per
  // slab counter fix_cnt, zeroed per launch) adds them in k order and stores the tile.
  int tail_u0, tail_parts, tail_kbpp;
  float* fix_ws;
  uint32_t* fix_cnt;
};

// ---------------------------------------------------------------- k-pacing (STORE GEMMs)
// Clusters that share A or B tiles (the 8-m-tile band order) only share them through L2 if
// they read the same k-slabs at about the same time.  Left free, persistent clusters drift
// apart over long K and the L2 working set outgrows 126 MB (measured: 57 GB of DRAM reads
// per 16384^3 launch vs ~2.6 GB at 8192^3), which costs power and hence clock.  Each CTA's
// producer therefore arrives at a global epoch counter every kSyncE k-blocks and, before
// loading epoch e, waits until every CTA has started epoch e - kSyncS: the grid stays within
// ~kSyncS epochs of k.  Counters live in the caller's workspace (kSyncR monotone slots,
// zeroed per launch); it is a throttle only -- results do not depend on it.
constexpr int kSyncE = 8;   // default k-blocks (of 64) per epoch
constexpr int kSyncS = 2;   // default slack in epochs (tools/pace_sweep.py)
constexpr int kSyncR = 8;   // counter ring (> slack)

__device__ __forceinline__ void sync_arrive(uint32_t* sync, uint32_t e) {
  atomicAdd(sync + (e % kSyncR), 1u);
}
// Returns false if the wait gave up: pacing assumes every CTA of the grid is resident (one
// persistent CTA per SM); if another kernel holds SMs and some CTAs have not started, the
// waiters stop pacing after kSyncTimeoutNs instead of deadlocking, and the kernel runs unpaced.
constexpr unsigned long long kSyncTimeoutNs = 200000ull;
__device__ __forceinline__ bool sync_wait(const uint32_t* sync, uint32_t e, uint32_t nctas) {
  const uint32_t need = nctas * (e / kSyncR + 1);
  const uint32_t* c = sync + (e % kSyncR);
  uint32_t v;
  const unsigned long long t0 = globaltimer_ns();
  while (true) {
    asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(c) : "memory");
    if ((int32_t)(v - need) >= 0) return true;
    if (globaltimer_ns() - t0 > kSyncTimeoutNs) return false;
    __nanosleep(64);
  }
}

template <int CG, int BN>
struct Geo {
  static constexpr int BNC = BN / CG;                  // B rows staged per CTA
  static constexpr int A_BYTES = kBM * kBK * 2;        // one of A_hi / A_lo
  static constexpr int B_BYTES = BNC * kBK * 2;        // one of B_hi / B_lo
  static constexpr int STAGE_BYTES = 2 * A_BYTES + 2 * B_BYTES;
};

// epilogue warps: NEPI in {8, 16}; NEPI/4 warps share each TMEM lane quarter and split
// its BN columns.  Kernel block = 4 control warps + NEPI epilogue warps.
template <int NEPI, bool FA = false>
struct EpiGeo {
  static constexpr int GPQ = NEPI / 4;            // column groups per lane quarter
  // FA (fused A split): one extra warpgroup of converter warps in front
  static constexpr int THREADS = (FA ? 256 : 128) + 32 * NEPI;
  static constexpr int W_PROD = FA ? 4 : 0;       // TMA producer
  static constexpr int W_MMA = FA ? 5 : 1;        // MMA issuer
  static constexpr int W_ALLOC = FA ? 6 : 2;      // TMEM allocator
  static constexpr int EPI0 = FA ? 8 : 4;         // first epilogue warp
};

struct UnitInfo {
  int m_tile, n_begin, n_count, slice;
  int kb0, kb1, ks;  // the unit's k-blocks [kb0, kb1) and split-K part (STORE); else [0, num_kb)
  int fx;            // STORE tail split: index of the unit's tile among the split tiles (else -1)
};

template <int EPI>
__device__ __forceinline__ UnitInfo decode_unit(const KParams& p, int u) {
  UnitInfo r;
  r.kb0 = 0;
  r.kb1 = p.num_kb;
  r.ks = 0;
  r.fx = -1;
  if constexpr (EPI == EPI_STORE) {
    // split-K (R21's k-parts): the parts of one tile are consecutive units
    if (p.ksplit > 1) {
      r.ks = u % p.ksplit;
      u /= p.ksplit;
      r.kb0 = r.ks * p.kb_per_part;
      r.kb1 = min(p.num_kb, r.kb0 + p.kb_per_part);
    } else if (p.tail_parts > 1 && u >= p.tail_u0) {
      // tail split: the k-parts of the last wave's tiles (consecutive units: concurrent)
      const int v = u - p.tail_u0;
      r.fx = v / p.tail_parts;
      r.ks = v - r.fx * p.tail_parts;
      r.kb0 = r.ks * p.tail_kbpp;
      r.kb1 = min(p.num_kb, r.kb0 + p.tail_kbpp);
      u = p.tail_u0 + r.fx;
    }
    // bands of up to band_m (8) m-tiles, m fastest inside a band: concurrent clusters share
    // A and B k-slabs in L2.
    const int GM = p.band_m;
    int band = u / (GM * p.n_tiles);
    int m0 = band * GM;
    int gm = min(GM, p.m_tiles - m0);
    int idx = u - band * GM * p.n_tiles;
    r.m_tile = m0 + idx % gm;
    r.n_begin = idx / gm;
    r.n_count = 1;
    r.slice = 0;
  } else if constexpr (EPI == EPI_KNN) {
    // concurrent clusters share the reference slice (B) -> one HBM read per B tile.
    r.slice = u / p.m_tiles;
    r.m_tile = u - r.slice * p.m_tiles;
    r.n_begin = r.slice * p.tiles_per_slice;
    r.n_count = min(p.tiles_per_slice, p.n_tiles - r.n_begin);
    if (r.n_count < 0) r.n_count = 0;
  } else {
    r.m_tile = u;
    r.n_begin = 0;
    r.n_count = p.n_tiles;
    r.slice = 0;
  }
  return r;
}

// lexicographic (key, idx) insertion into an ascending register list of length KN
template <int KN>
__device__ __forceinline__ void topk_insert(float (&kd)[KN], int (&ki)[KN], float key, int idx) {
  if (key < kd[KN - 1] || (key == kd[KN - 1] && idx < ki[KN - 1])) {
    kd[KN - 1] = key;
    ki[KN - 1] = idx;
#pragma unroll
    for (int t = KN - 1; t > 0; t--) {
      bool sw = (kd[t] < kd[t - 1]) || (kd[t] == kd[t - 1] && ki[t] < ki[t - 1]);
      float a = kd[t], b = kd[t - 1];
      int ia = ki[t], ib = ki[t - 1];
      kd[t] = sw ? b : a;
      kd[t - 1] = sw ? a : b;
      ki[t] = sw ? ib : ia;
      ki[t - 1] = sw ? ia : ib;
    }
  }
}

// streaming insertion (indices arrive in increasing order): strict '<' is enough.  All 16
// comparisons against the old list are independent (c_t = key < kd[t], monotone in t), and
// each slot takes its left neighbour (c_{t-1}), the new key (c_t only) or itself: no serial
// compare-swap chain, so the insertion costs ~5 dependent ALU latencies instead of ~48.
template <int KN>
__device__ __forceinline__ void topk_insert_stream(float (&kd)[KN], int (&ki)[KN], float key,
                                                   int idx) {
  bool c[KN];
#pragma unroll
  for (int t = 0; t < KN; t++) c[t] = key < kd[t];
#pragma unroll
  for (int t = KN - 1; t > 0; t--) {
    kd[t] = c[t - 1] ? kd[t - 1] : (c[t] ? key : kd[t]);
    ki[t] = c[t - 1] ? ki[t - 1] : (c[t] ? idx : ki[t]);
  }
  kd[0] = c[0] ? key : kd[0];
  ki[0] = c[0] ? idx : ki[0];
}

__device__ __forceinline__ void named_bar_sync(int id, int nthreads) {
  asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(nthreads) : "memory");
}


// y = h + m + l exactly, each part with <= 11 significant bits and its 13 low mantissa bits
// zero, i.e. exact tf32 operands (kind::tf32 ignores those bits).  Truncation split: h keeps
// y's top 11 bits, r = y - h (exact) its low 13, m the top 11 of r, l = r - m (exact, <= 2).
__device__ __forceinline__ void tf32_parts(float y, float& h, float& m, float& l) {
  h = __uint_as_float(__float_as_uint(y) & 0xFFFFE000u);
  const float r = __fsub_rn(y, h);
  m = __uint_as_float(__float_as_uint(r) & 0xFFFFE000u);
  l = __fsub_rn(r, m);
}

template <int CG, int BN, bool SEP, int EPI, int STAGES, int NEPI, bool FA, bool AR, bool AS, bool FB,
          int KN>
__global__ void __launch_bounds__(EpiGeo<NEPI, FA || FB>::THREADS, 1)
    egemm_tc_kernel(const __grid_constant__ CUtensorMap tm_ahi,
                    const __grid_constant__ CUtensorMap tm_alo,
                    const __grid_constant__ CUtensorMap tm_bhi,
                    const __grid_constant__ CUtensorMap tm_blo,
                    const __grid_constant__ CUtensorMap tm_d, const KParams p) {
  using G = Geo<CG, BN>;
  // FB (fused B split): the converter warpgroup builds B_hi / B_lo from TMA-staged fp32 B
  // tiles (row-major K x N, transposed to K-major on the way) while A comes pre-split by TMA
  constexpr bool CONV = FA || FB;
  using EG = EpiGeo<NEPI, CONV>;
  constexpr int GPQ = EG::GPQ;
  constexpr int COLS = BN / GPQ;  // columns per epilogue warp
  constexpr int NACC = SEP ? 4 : 2;
  constexpr uint32_t TMEM_COLS = (NACC * BN <= 32) ? 32 : (NACC * BN <= 64) ? 64
                                 : (NACC * BN <= 128) ? 128 : (NACC * BN <= 256) ? 256 : 512;
  static_assert(NACC * BN <= 512, "TMEM overflow");
  static_assert(!(EPI != EPI_STORE && SEP), "kNN / kMeans: single accumulator (norm MMA)");
  static_assert(COLS % 32 == 0 || (EPI == EPI_STORE && COLS % 16 == 0), "epilogue column split");
  // TMEM -> register load width of the STORE epilogue (BN = 224: 112 columns per warp)
  constexpr int LDW = (COLS % 32 == 0) ? 32 : 16;

  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) &
                                             ~uintptr_t(1023));
  // AR (A resident, kNN / kMeans with K <= 128): the A tile of a unit is loaded once into
  // its own buffer and the ring carries only B; otherwise each stage holds A and B.
  // NORM (kNN / kMeans): each stage also has a 32-B row per staged B row for the tf32 norm
  // parts (written by the norm warp on a tile's last k-block), plus one A' tile of ones.
  constexpr bool NORM = (EPI != EPI_STORE);
  // KREG (kNN, 8 epilogue warps): a thread's whole column share of a tile (COLS fp32) is
  // loaded from TMEM at once and the accumulator handed back before any of it is ranked, so
  // the top-k work of tile t overlaps the MMAs of tiles t+1 and t+2; the registers come from
  // the control warpgroup (setmaxnreg 56 / 216: 4x32x56 + 8x32x216 <= 64K).
  constexpr bool KREG = (EPI == EPI_KNN) && AR && !FA && NEPI == 8 && COLS == 128 && KN == 16;
  // kNN lists longer than 16 (k <= 32 / 64): the per-32-column path with the registers of
  // the control warpgroup (setmaxnreg 56 / 216), no software-pipelined TMEM loads
  constexpr bool BIGREG = KREG || (EPI == EPI_KNN && KN > 16 && !CONV);
  static_assert(KN == 16 || KN == 32 || KN == 64, "kNN list length");
  constexpr int NP_OFF = AR ? 2 * G::B_BYTES : G::STAGE_BYTES;  // norm parts inside a stage
  constexpr int NP_BYTES = NORM ? G::BNC * 32 : 0;
  constexpr int SB = NP_OFF + NP_BYTES;                       // bytes per ring stage
  constexpr int B_OFF = AR ? 0 : 2 * G::A_BYTES;            // B_hi offset inside a stage
  constexpr int AR_BYTES = AR ? 2 * 2 * G::A_BYTES : 0;     // 2 k-blocks of A_hi + A_lo
  constexpr int ONES_BYTES = NORM ? kBM * 32 : 0;
  static_assert(SB % 1024 == 0, "stage alignment");
  // AS (fused A, TMA-staged): the fp32 A tiles land in their own ring (NSTG x 128 rows x 64
  // fp32, two 128-B-swizzled boxes of 32 columns), loaded ahead by warp 7; the converters
  // split from smem instead of waiting on their own global loads.
  // AS: the fp32 A tile (32 KiB = the A_hi + A_lo bytes of a stage) lands in the stage's own A
  // region and the converters split it in place; FB keeps a 3-slot fp32 staging ring.
  constexpr int NSTG = FB ? 3 : 0;
  constexpr int STG_BYTES = kBM * kBK * 4;
  static_assert(!AS || FA, "AS is a fused-A mode");
  static_assert(!(FA && FB), "one fused operand at a time");
  static_assert(!FB || (CG == 2 && (BN == 256 || BN == 224) && EPI == EPI_STORE && !SEP),
                "FB: 256 x 256 or 256 x 224 pair tiles");
  uint8_t* stage_base = smem;
  uint8_t* a_res = smem + STAGES * SB;
  uint8_t* a_stg = a_res + AR_BYTES;
  uint8_t* ones_tile = a_stg + NSTG * STG_BYTES;
  uint64_t* bars = reinterpret_cast<uint64_t*>(ones_tile + ONES_BYTES);
  uint64_t* full = bars;
  uint64_t* empty = bars + STAGES;
  uint64_t* acc_full = bars + 2 * STAGES;
  uint64_t* acc_empty = bars + 2 * STAGES + 2;
  // AR: resident A slots (K <= 64: two slots, the next unit's tile loads while this unit's
  // MMAs run; K <= 128: one slot holding both k-blocks)
  uint64_t* a_full = bars + 2 * STAGES + 4;
  uint64_t* a_empty = bars + 2 * STAGES + 5;
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(bars + 2 * STAGES + 6);
  uint64_t* a_full1 = bars + 2 * STAGES + 7;
  uint64_t* a_empty1 = bars + 2 * STAGES + 8;
  uint64_t* sfull = bars + 2 * STAGES + 10;  // AS: fp32 A tile landed (TMA bytes)
  uint64_t* sempty = sfull + NSTG;           // AS: consumed by the 4 converter warps
  uint64_t* afull = sempty + NSTG;           // AS: a stage's fp32 A tile landed (TMA bytes)
  uint8_t* scratch = reinterpret_cast<uint8_t*>(bars + 2 * STAGES + 10 + 2 * NSTG + (AS ? STAGES : 0));  // merges
  // TS (STORE): the result leaves through TMA stores -- each epilogue warp stages a 32 x 32
  // fp32 block (128-B rows, 128-B swizzle) in its own 4 KiB buffer and one lane issues a
  // bulk tensor store: coalesced full-line writes, the LSU free for the next unit's drains
  // (the per-lane row stores wrote 32 rows x 16 B per instruction)
  constexpr bool TS = (EPI == EPI_STORE) && !FB && (COLS % 32 == 0);
  const uint32_t ts_base = (ptx::smem_u32(scratch) + 1023u) & ~1023u;

  const int warp = threadIdx.x >> 5;
  const int lane = threadIdx.x & 31;
  const uint32_t rank = (CG == 2) ? ptx::cluster_ctarank() : 0u;
  const int cluster = (CG == 2) ? (int)ptx::cluster_id_x() : (int)blockIdx.x;
  const int nclusters = (CG == 2) ? (int)ptx::nclusters_x() : (int)gridDim.x;
  const bool leader = (rank == 0);
  if (threadIdx.x == 0) {
    TL(0);
    if (DIAG_MODE(2048) && blockIdx.x == 0) p.probe[8 + 10] = globaltimer_ns();
  }

  if (warp == EG::W_PROD && lane == 0) {
    ptx::prefetch_tmap(&tm_ahi);  // (FA: tm_ahi maps the fp32 A: staged loads / L2 prefetch)
    if (!FA) ptx::prefetch_tmap(&tm_alo);  // (FB: tm_bhi maps the fp32 B, tm_blo a copy)
    ptx::prefetch_tmap(&tm_bhi);
    ptx::prefetch_tmap(&tm_blo);
  }
  if (warp == EG::W_MMA && lane == 0) {
    for (int s = 0; s < STAGES; s++) {
      // FA: the producer's expect_tx arrive plus one arrive per converter warp of the pair;
      // NORM: plus one arrive per norm warp of the pair
      ptx::mbar_init(&full[s], 1 + (CONV ? 4 * CG : 0) + (NORM ? CG : 0));
      ptx::mbar_init(&empty[s], 1);
    }
    for (int b = 0; b < 2; b++) {
      ptx::mbar_init(&acc_full[b], 1);
      ptx::mbar_init(&acc_empty[b], NEPI * CG);  // one arrive per epilogue warp of the pair
    }
    ptx::mbar_init(a_full, 1);
    ptx::mbar_init(a_empty, 1);
    ptx::mbar_init(a_full1, 1);
    ptx::mbar_init(a_empty1, 1);
    if constexpr (AS)
      for (int s = 0; s < STAGES; s++) ptx::mbar_init(&afull[s], 1);
    for (int i = 0; i < NSTG; i++) {
      ptx::mbar_init(&sfull[i], 1);
      ptx::mbar_init(&sempty[i], 4);
    }
    ptx::fence_mbar_init();
  }
  if (!FA && !AR && DIAG_NO_TMA && DIAG_MODE(32)) {
    // diagnostics only: fill the ring with random fp16 operands (hi ~[0.5, 1), lo ~2^-9) so a
    // NO_TMA run multiplies realistic data -- isolates the power of the operand traffic
    for (int i = threadIdx.x; i < STAGES * SB / 16; i += blockDim.x) {
      const int off = (i * 16) % SB;
      const bool lo_part = (off >= G::A_BYTES && off < 2 * G::A_BYTES) || off >= 2 * G::A_BYTES + G::B_BYTES;
      uint32_t w[4];
#pragma unroll
      for (int j = 0; j < 4; j++) {
        uint32_t h = (uint32_t)(i * 4 + j + 1) * 2654435761u + blockIdx.x * 40503u;
        h ^= h >> 15; h *= 2246822519u; h ^= h >> 13;
        const uint32_t e = lo_part ? 0x1800u : 0x3800u;
        w[j] = ((h & 0x83FFu) | e) | ((((h >> 16) & 0x83FFu) | e) << 16);
      }
      ptx::sts128(ptx::smem_u32(stage_base) + i * 16, w[0], w[1], w[2], w[3]);
    }
    ptx::fence_proxy_async_smem();
  }
  if constexpr (NORM) {
    if (warp == 3) {
      // A' = rows of (1, 1, 1, 0) in both 16-B chunks of every 32-B row: invariant under the
      // 32-B swizzle's chunk exchange, so B' may hold its parts in either chunk.  The NP
      // slots start zeroed; the norm warp later rewrites only the parts chunk of a row.
      const uint32_t o = ptx::smem_u32(ones_tile);
      for (int i = lane; i < ONES_BYTES / 16; i += 32) ptx::sts128f(o + i * 16, 1.f, 1.f, 1.f, 0.f);
      for (int st = 0; st < STAGES; st++) {
        const uint32_t np = ptx::smem_u32(stage_base + st * SB + NP_OFF);
        for (int i = lane; i < NP_BYTES / 16; i += 32) ptx::sts128f(np + i * 16, 0.f, 0.f, 0.f, 0.f);
      }
      ptx::fence_proxy_async_smem();
    }
  }
  if (warp == EG::W_ALLOC) ptx::tmem_alloc<CG>(tmem_slot, TMEM_COLS);
  ptx::tc_fence_before();
  // (CG == 2: the cluster barrier orders the pair; the CTA barrier after it adds nothing but
  // lets compute-sanitizer's racecheck, which does not model barrier.cluster, see the order)
  if constexpr (CG == 2) { ptx::cluster_sync(); __syncthreads(); } else __syncthreads();
  ptx::tc_fence_after();
  const uint32_t tmem_base = *tmem_slot;
  // Every launch is a programmatic dependent of the previous kernel in the stream (the split
  // of this call, or anything else): the setup above ran under that kernel's tail; nothing
  // global is touched before it has completed.  (A peeled tail launch instead overlaps the
  // main grid of the same call -- disjoint rows -- and waits at its end.)
  if (!p.pdl_wait) asm volatile("griddepcontrol.wait;" ::: "memory");
  if (threadIdx.x == 0) TL(1);
  // STORE: a tail launch of the same call (the peeled last wave, launched with programmatic
  // stream serialisation) may start on the SMs this grid frees as its CTAs finish
  if (EPI == EPI_STORE && threadIdx.x == 0) asm volatile("griddepcontrol.launch_dependents;");
  if (blockIdx.x == 0 && threadIdx.x == 0 && !p.pdl_wait) {  // SM-clock probe (egemm_debug_last_clock)
    p.probe[0] = clock64();
    p.probe[1] = globaltimer_ns();
  }


  // FA register budget per warpgroup (512 threads share 64K registers): converters 96,
  // producer / MMA / allocator 56, the two epilogue warpgroups 176 (running totals).  Each
  // setmaxnreg sits at the top of its warpgroup's branch so it dominates that role's code.
  if (CONV && warp < 4) {
    if constexpr (CONV) asm volatile("setmaxnreg.dec.sync.aligned.u32 96;");
    if constexpr (FB) {
      // ================= fused round-split of B (converter warpgroup) =================
      // Alg. 1 l.3 for B inside the GEMM.  The fp32 tile of this CTA's BNC
      // (128 or 112) B columns x 64 k (one unswizzled TMA box, rows of k contiguous) sits in
      // the staging ring; thread t takes column n = t, reads its 8 k-chunks down the rows
      // (a warp reads 32 consecutive words of one row per instruction: conflict-free), splits
      // them and stores 16-B hi / lo chunks into row n of the K-major 128-B-swizzled B stage.
      int stage = 0;
      uint32_t phase = 0;
      int si = 0;
      uint32_t sph = 0;
      const int n = threadIdx.x;  // 0 .. 127 (columns >= BNC idle)
      constexpr int ROWB = G::BNC * 4;  // bytes per staged k-row
      const bool act = n < G::BNC;
      for (int u = cluster; u < p.num_units; u += nclusters) {
        UnitInfo ui = decode_unit<EPI>(p, u);
        for (int ns = 0; ns < ui.n_count; ns++) {
          for (int kb = ui.kb0; kb < ui.kb1; kb++) {
            ptx::mbar_wait(&sfull[si], sph);
            ptx::mbar_wait(&empty[stage], phase ^ 1u);
            const uint32_t sb = ptx::smem_u32(stage_base + stage * G::STAGE_BYTES) + 2 * G::A_BYTES;
            const uint32_t xb = ptx::smem_u32(a_stg + si * STG_BYTES) + 4 * n;
#pragma unroll
            for (int c = 0; c < kBK / 8; c++) {
              if (!act) break;
              float x[8];
#pragma unroll
              for (int i = 0; i < 8; i++) x[i] = ptx::lds32f(xb + (c * 8 + i) * ROWB);  // k = 8c + i
              uint32_t hi[4], lo[4];
#pragma unroll
              for (int e = 0; e < 4; e++) ptx::split2(x[2 * e], x[2 * e + 1], hi[e], lo[e]);
              const uint32_t off = (uint32_t)(n * 128 + ((c ^ (n & 7)) << 4));
              ptx::sts128(sb + off, hi[0], hi[1], hi[2], hi[3]);
              ptx::sts128(sb + G::B_BYTES + off, lo[0], lo[1], lo[2], lo[3]);
            }
            ptx::fence_proxy_async_smem();  // generic-proxy stores -> visible to tcgen05.mma
            __syncwarp();
            if (lane == 0) {
              ptx::mbar_arrive_cluster(&full[stage], 0);
              ptx::mbar_arrive(&sempty[si]);
            }
            if (++stage == STAGES) { stage = 0; phase ^= 1u; }
            if (++si == NSTG) { si = 0; sph ^= 1u; }
          }
        }
      }
    }
    // ================= fused round-split of A (converter warpgroup) =================
    // Alg. 1 l.2 inside the GEMM: each thread loads 8 consecutive fp32 of one
    // A row (2 x 16 B), splits them (cvt.rn) and stores the 16 B hi / lo chunks straight
    // into the 128-B-swizzled K-major stage layout the MMA descriptors expect -- the
    // paper's LDG -> register -> STS staging with the split folded in.
    if constexpr (FA) {
      int stage = 0;
      uint32_t phase = 0;
      int si = 0;          // AS: staging ring slot / parity
      uint32_t sph = 0;
      int conv_n = 0;  // (diagnostics: timeline slot 8)
      const int c = lane & 7;         // 16-B chunk (8 fp16) of the 128-B row
      const int rsub = lane >> 3;     // 4 rows per warp instruction
      for (int u = cluster; u < p.num_units; u += nclusters) {
        UnitInfo ui = decode_unit<EPI>(p, u);
        const int64_t arow0 = (int64_t)ui.m_tile * (kBM * CG) + rank * kBM;
        for (int ns = 0; ns < ui.n_count; ns++) {
          for (int kb = ui.kb0; kb < ui.kb1; kb++) {
            if constexpr (AS) {
              // the stage's A region holds the fp32 tile (2 boxes of 32 columns, SW128): row r,
              // 8 values k = 8c..8c+7 are fp32 16-B chunks 2(c%4), 2(c%4)+1 of box c/4 at chunk
              // position j ^ (r & 7).  Each converter warp reads its 32 rows' values, then
              // overwrites them with the hi / lo K-major tiles: the hi rows of warp w land on
              // box 0's rows of warp w, the lo rows on box 1's -- a warp only overwrites what it
              // has itself read (in order within the warp), so the warps need no barrier.
              ptx::mbar_wait(&afull[stage], phase);  // (the producer waited for the free stage)
              const uint32_t sb = ptx::smem_u32(stage_base + stage * G::STAGE_BYTES);
              const uint32_t xb = sb + (c >> 2) * (STG_BYTES / 2);
              const int j0 = (c & 3) * 2;
              if (DIAG_MODE(4096)) {  // diagnostics only: hand the fp32 tile over unconverted
                if (lane == 0) {      // (results wrong by design: bounds the conversion's cost)
                  if constexpr (CG == 1) ptx::mbar_arrive(&full[stage]);
                  else ptx::mbar_arrive_cluster(&full[stage], 0);
                }
                if (++stage == STAGES) { stage = 0; phase ^= 1u; }
                continue;
              }
              float4 u[16];
#pragma unroll
              for (int it = 0; it < 8; it++) {
                const int r = warp * 32 + it * 4 + rsub;
                const uint32_t rb = xb + r * 128;
                u[2 * it] = ptx::lds128f(rb + ((j0 ^ (r & 7)) << 4));
                u[2 * it + 1] = ptx::lds128f(rb + (((j0 + 1) ^ (r & 7)) << 4));
              }
              __syncwarp();  // this warp's fp32 values are in registers
#pragma unroll
              for (int it = 0; it < 8; it++) {
                const int r = warp * 32 + it * 4 + rsub;
                uint32_t hi[4], lo[4];
                ptx::split2(u[2 * it].x, u[2 * it].y, hi[0], lo[0]);
                ptx::split2(u[2 * it].z, u[2 * it].w, hi[1], lo[1]);
                ptx::split2(u[2 * it + 1].x, u[2 * it + 1].y, hi[2], lo[2]);
                ptx::split2(u[2 * it + 1].z, u[2 * it + 1].w, hi[3], lo[3]);
                const uint32_t off = (uint32_t)(r * 128 + ((c ^ (r & 7)) << 4));
                ptx::sts128(sb + off, hi[0], hi[1], hi[2], hi[3]);
                ptx::sts128(sb + G::A_BYTES + off, lo[0], lo[1], lo[2], lo[3]);
              }
              ptx::fence_proxy_async_smem();  // generic-proxy stores -> visible to tcgen05.mma
              __syncwarp();
              if (lane == 0) {
                if constexpr (CG == 1) ptx::mbar_arrive(&full[stage]);
                else ptx::mbar_arrive_cluster(&full[stage], 0);
                if (warp == 0 && conv_n++ == 0) TL(8);
              }
              if (++stage == STAGES) { stage = 0; phase ^= 1u; }
              continue;
            }
            ptx::mbar_wait(&empty[stage], phase ^ 1u);
            const uint32_t sb = ptx::smem_u32(stage_base + stage * G::STAGE_BYTES);
            const int k = kb * kBK + c * 8;
            float4 x[16];
#pragma unroll
            for (int it = 0; it < 8; it++) {
              const int r = warp * 32 + it * 4 + rsub;
              const int64_t row = arow0 + r;
              const float* src = p.a_f32 + row * p.lda_f32 + k;
              if (row < p.M && k + 8 <= p.K && p.vec_a) {
                x[2 * it] = __ldg(reinterpret_cast<const float4*>(src));
                x[2 * it + 1] = __ldg(reinterpret_cast<const float4*>(src + 4));
              } else {
                float t[8];
#pragma unroll
                for (int e = 0; e < 8; e++) t[e] = (row < p.M && k + e < p.K) ? __ldg(src + e) : 0.f;
                x[2 * it] = make_float4(t[0], t[1], t[2], t[3]);
                x[2 * it + 1] = make_float4(t[4], t[5], t[6], t[7]);
              }
            }
#pragma unroll
            for (int it = 0; it < 8; it++) {
              const int r = warp * 32 + it * 4 + rsub;
              uint32_t hi[4], lo[4];
              const float* f = reinterpret_cast<const float*>(&x[2 * it]);
#pragma unroll
              for (int e = 0; e < 4; e++) ptx::split2(f[2 * e], f[2 * e + 1], hi[e], lo[e]);
              const uint32_t off = (uint32_t)(r * 128 + ((c ^ (r & 7)) << 4));
              ptx::sts128(sb + off, hi[0], hi[1], hi[2], hi[3]);
              ptx::sts128(sb + G::A_BYTES + off, lo[0], lo[1], lo[2], lo[3]);
            }
            ptx::fence_proxy_async_smem();  // generic-proxy stores -> visible to tcgen05.mma
            __syncwarp();
            if (lane == 0) {
              if constexpr (CG == 1) ptx::mbar_arrive(&full[stage]);
              else ptx::mbar_arrive_cluster(&full[stage], 0);
            }
            if (++stage == STAGES) { stage = 0; phase ^= 1u; }
          }
        }
      }
    }
  } else if (warp < EG::EPI0) {
   if constexpr (CONV || BIGREG) asm volatile("setmaxnreg.dec.sync.aligned.u32 56;");
   if (warp == EG::W_PROD) {
    // ============================ TMA producer ============================
    if (lane == 0) {
      TL(15);
      int stage = 0;
      uint32_t phase = 0;
      // FA: only B comes through TMA (A is written by the converter warps); AR: the ring
      // carries only B, A is loaded once per unit into a_res
      constexpr uint32_t TX = (FA || AR) ? 2 * G::B_BYTES : FB ? 2 * G::A_BYTES : G::STAGE_BYTES;
      uint32_t uctr = 0;
      const bool pace = (EPI == EPI_STORE) && p.sync != nullptr && !DIAG_NO_TMA;
      bool pace_wait = pace;
      uint32_t gkb = 0;  // k-blocks this CTA has started loading, over all its units
      const bool idle = DIAG_NO_TMA && DIAG_MODE(2);  // diagnostics only
      for (int u = idle ? p.num_units : cluster; u < p.num_units; u += nclusters, uctr++) {
        UnitInfo ui = decode_unit<EPI>(p, u);
        const int arow = ui.m_tile * (kBM * CG) + (int)rank * kBM;
        if constexpr (AR) {
          const uint32_t nsl = p.num_kb == 1 ? 2u : 1u, slot = uctr % nsl, use = uctr / nsl;
          uint64_t* af = slot ? a_full1 : a_full;
          ptx::mbar_wait(slot ? a_empty1 : a_empty, (use & 1u) ^ 1u);  // the slot's last unit is done
          if (leader) ptx::mbar_arrive_expect_tx(af, 2 * G::A_BYTES * p.num_kb * CG);
          for (int kb = 0; kb < p.num_kb; kb++) {
            uint8_t* ab = a_res + (slot + kb) * 2 * G::A_BYTES;
            if constexpr (CG == 1) {
              ptx::tma_load_2d(&tm_ahi, af, ab, kb * kBK, arow);
              ptx::tma_load_2d(&tm_alo, af, ab + G::A_BYTES, kb * kBK, arow);
            } else {
              ptx::tma_load_2d_pair(&tm_ahi, af, ab, kb * kBK, arow);
              ptx::tma_load_2d_pair(&tm_alo, af, ab + G::A_BYTES, kb * kBK, arow);
            }
          }
        }
        for (int ns = 0; ns < ui.n_count; ns++) {
          const int brow = (ui.n_begin + ns) * BN + (int)rank * G::BNC;
          for (int kb = ui.kb0; kb < ui.kb1; kb++) {
            if (pace && (gkb % (uint32_t)p.pace_e) == 0) {
              const uint32_t e = gkb / (uint32_t)p.pace_e;
              sync_arrive(p.sync, e);
              // a wait that times out (not all CTAs resident) stops this CTA's waiting but not
              // its arrivals, so the CTAs that do pace are never held up by it
              if (pace_wait && e >= (uint32_t)p.pace_s && !sync_wait(p.sync, e - p.pace_s, gridDim.x))
                pace_wait = false;
            }
            gkb++;
            if (FA && p.a_pf && ns == 0) {
              // the fp32 A tile a_pf k-blocks ahead into L2 (TMA bulk prefetch: no smem),
              // continuing into this CTA's next unit near the end of a unit, so the
              // converters' loads (LDG, or the staged TMA copies) hit L2 instead of DRAM
              auto pf = [&](int kbp, int row) {
                ptx::tma_prefetch_2d_l2(&tm_ahi, kbp * kBK, row);
                if (AS) ptx::tma_prefetch_2d_l2(&tm_ahi, kbp * kBK + kBK / 2, row);  // 32-column boxes
              };
              if (kb == ui.kb0 && uctr == 0)
                for (int j = ui.kb0; j < ui.kb0 + p.a_pf && j < ui.kb1; j++) pf(j, arow);
              const int kf = kb + p.a_pf;
              if (kf < ui.kb1) {
                pf(kf, arow);
              } else if (u + nclusters < p.num_units) {
                const UnitInfo nu = decode_unit<EPI>(p, u + nclusters);
                if (nu.kb0 + kf - ui.kb1 < nu.kb1)
                  pf(nu.kb0 + kf - ui.kb1, nu.m_tile * (kBM * CG) + (int)rank * kBM);
              }
            }
            ptx::mbar_wait(&empty[stage], phase ^ 1u);
            uint8_t* sb = stage_base + stage * SB;
            if (DIAG_NO_TMA) {  // diagnostics only: MMA-issue ceiling without operand traffic
              if (leader && !CONV) ptx::mbar_arrive(&full[stage]);
              if (++stage == STAGES) { stage = 0; phase ^= 1u; }
              continue;
            }
            // (diagnostics only, bit 1024: after the ring's first fill, skip the B loads -- the
            // MMAs re-read real but stale B tiles; the time / clock change bounds what removing
            // B's L2 -> smem traffic can buy)
            const bool skip_b = DIAG_MODE(1024) && (FA || AR) && gkb > (uint32_t)STAGES;
            if (leader) {
              if (skip_b) ptx::mbar_arrive(&full[stage]);
              else ptx::mbar_arrive_expect_tx(&full[stage], TX * CG);
            }
            const int k0 = kb * kBK;
            if (gkb == 1) TL(14);
            if constexpr (AS) {  // this CTA's fp32 A tile into the stage's A region
              ptx::mbar_arrive_expect_tx(&afull[stage], STG_BYTES);
              ptx::tma_load_2d(&tm_ahi, &afull[stage], sb, k0, arow);
              ptx::tma_load_2d(&tm_ahi, &afull[stage], sb + STG_BYTES / 2, k0 + 32, arow);
            }
            if constexpr (CG == 1) {
              if (!FA && !AR) {
                ptx::tma_load_2d(&tm_ahi, &full[stage], sb, k0, arow);
                ptx::tma_load_2d(&tm_alo, &full[stage], sb + G::A_BYTES, k0, arow);
              }
              if (!FB && !skip_b) {
                ptx::tma_load_2d(&tm_bhi, &full[stage], sb + B_OFF, k0, brow);
                ptx::tma_load_2d(&tm_blo, &full[stage], sb + B_OFF + G::B_BYTES, k0, brow);
              }
            } else {
              if (!FA && !AR) {
                ptx::tma_load_2d_pair(&tm_ahi, &full[stage], sb, k0, arow);
                ptx::tma_load_2d_pair(&tm_alo, &full[stage], sb + G::A_BYTES, k0, arow);
              }
              if (!FB && !skip_b) {
                ptx::tma_load_2d_pair(&tm_bhi, &full[stage], sb + B_OFF, k0, brow);
                ptx::tma_load_2d_pair(&tm_blo, &full[stage], sb + B_OFF + G::B_BYTES, k0, brow);
              }
            }
            if (gkb == 1) TL(2);
            if (++stage == STAGES) { stage = 0; phase ^= 1u; }
          }
        }
      }
      if (pace) {  // out of units: arrive at every remaining epoch so nobody waits on us
        const uint32_t per_cta = (uint32_t)((p.num_units + nclusters - 1) / nclusters) *
                                 (uint32_t)(p.ksplit > 1 ? p.kb_per_part : p.num_kb);
        const uint32_t pe = (uint32_t)p.pace_e;
        const uint32_t total = (per_cta + pe - 1) / pe;
        for (uint32_t e = (gkb + pe - 1) / pe; e < total; e++) sync_arrive(p.sync, e);
      }
    }
  } else if (FB && warp == 7) {
    // ==================== fp32 B staging producer (fused B) ====================
    if constexpr (FB) {
      if (lane == 0) {
        int si = 0;
        uint32_t sph = 0;
        for (int u = cluster; u < p.num_units; u += nclusters) {
          UnitInfo ui = decode_unit<EPI>(p, u);
          for (int ns = 0; ns < ui.n_count; ns++) {
            const int n0 = (ui.n_begin + ns) * BN + (int)rank * G::BNC;
            for (int kb = ui.kb0; kb < ui.kb1; kb++) {
              ptx::mbar_wait(&sempty[si], sph ^ 1u);
              ptx::mbar_arrive_expect_tx(&sfull[si], G::BNC * kBK * 4);
              uint8_t* dst = a_stg + si * STG_BYTES;
              ptx::tma_load_2d(&tm_bhi, &sfull[si], dst, n0, kb * kBK);
              if (++si == NSTG) { si = 0; sph ^= 1u; }
            }
          }
        }
      }
    }
  } else if (NORM && warp == 3) {
    // ============================ norm warp (kNN / kMeans) ============================
    // Follows the stage ring; on a tile's last k-block writes, for each of this CTA's BNC
    // staged B rows j, the tf32 parts of y_j = -||b_j||^2 / 2 (columns >= N: 0) into the
    // stage's norm slot, then arrives on the stage's full barrier like the TMA bytes do.
    if constexpr (NORM) {
      int stage = 0;
      uint32_t phase = 0;
      for (int u = cluster; u < p.num_units; u += nclusters) {
        UnitInfo ui = decode_unit<EPI>(p, u);
        for (int ns = 0; ns < ui.n_count; ns++) {
          const int64_t brow0 = (int64_t)(ui.n_begin + ns) * BN + (int)rank * G::BNC;
          for (int kb = ui.kb0; kb < ui.kb1; kb++) {
            ptx::mbar_wait(&empty[stage], phase ^ 1u);
            if (kb == p.num_kb - 1) {
              const uint32_t np = ptx::smem_u32(stage_base + stage * SB + NP_OFF);
#pragma unroll
              for (int j = 0; j < G::BNC / 32; j++) {
                const int r = j * 32 + lane;  // lane-contiguous 32-B rows: conflict-free
                const int64_t col = brow0 + r;
                const float bn = col < p.N ? __ldg(p.bnorm + col) : 0.f;
                float h, m, l;
                tf32_parts(-0.5f * bn, h, m, l);  // -bn/2 is exact
                ptx::sts128f(np + r * 32, h, m, l, 0.f);
              }
              ptx::fence_proxy_async_smem();  // generic-proxy stores -> visible to tcgen05.mma
            }
            __syncwarp();
            if (lane == 0) {
              if constexpr (CG == 1) ptx::mbar_arrive(&full[stage]);
              else ptx::mbar_arrive_cluster(&full[stage], 0);
            }
            if (++stage == STAGES) { stage = 0; phase ^= 1u; }
          }
        }
      }
    }
  } else if (warp == EG::W_MMA) {
    // ============================ MMA issuer ============================
    // The whole warp runs the loop (so stage / descriptor arithmetic stays in uniform
    // registers); one elected lane -- always the same one -- issues MMAs and commits.
    if (leader) {
      // operand format: fp16 parts (the paper's round-split) or bf16 parts (NEXT-3 variant)
      const uint32_t idesc = ptx::idesc_f16_f32(kBM * CG, BN) | (p.bf16 ? ((1u << 7) | (1u << 10)) : 0u);
      const uint32_t sbase = ptx::smem_u32(stage_base);
      int stage = 0;
      uint32_t phase = 0;
      uint32_t chunk_ctr = 0;
      uint32_t uctr = 0;
      const uint32_t abase = ptx::smem_u32(a_res);
      for (int u = cluster; u < p.num_units; u += nclusters, uctr++) {
        UnitInfo ui = decode_unit<EPI>(p, u);
        const uint32_t nsl = p.num_kb == 1 ? 2u : 1u, aslot = AR ? uctr % nsl : 0u;
        if constexpr (AR) {
          ptx::mbar_wait(aslot ? a_full1 : a_full, (uctr / nsl) & 1u);  // this unit's A tile is resident
          ptx::tc_fence_after();
        }
        for (int ns = 0; ns < ui.n_count; ns++) {
          const int nch = (ui.kb1 - ui.kb0 + p.kb_per_chunk - 1) / p.kb_per_chunk;
          for (int ch = 0; ch < nch; ch++) {
            const uint32_t buf = chunk_ctr & 1u;
            const uint32_t use = chunk_ctr >> 1;
            ptx::mbar_wait(&acc_empty[buf], (use & 1u) ^ 1u);
            ptx::tc_fence_after();
            const uint32_t acc_hh = tmem_base + (SEP ? 2 * buf : buf) * BN;
            const uint32_t acc_x = SEP ? acc_hh + BN : acc_hh;
            const int kb0 = ui.kb0 + ch * p.kb_per_chunk;
            const int kb1 = min(ui.kb1, kb0 + p.kb_per_chunk);
            for (int kb = kb0; kb < kb1; kb++) {
              if (!(DIAG_NO_TMA && DIAG_MODE(2))) ptx::mbar_wait(&full[stage], phase);
              ptx::tc_fence_after();
              const uint32_t sa = sbase + stage * SB;
              const uint32_t aa = AR ? abase + (aslot + kb) * 2 * G::A_BYTES : sa;
              const uint64_t d_ahi = ptx::sdesc_kmajor_sw128(aa);
              const uint64_t d_alo = ptx::sdesc_kmajor_sw128(aa + G::A_BYTES);
              const uint64_t d_bhi = ptx::sdesc_kmajor_sw128(sa + B_OFF);
              const uint64_t d_blo = ptx::sdesc_kmajor_sw128(sa + B_OFF + G::B_BYTES);
              // Alg. 1 on every 16-wide k-slice, in the paper's order:
              // [lo*lo,] lo*hi, hi*lo, hi*hi chained through the accumulator (SEP: hi*hi in
              // its own).  The first MMA of a promotion chunk starts it from zero.
              const uint32_t acc0 = (kb > kb0) ? 1u : 0u;
              if (ptx::elect_one()) {
                // The lo*lo term is a separate branch, not a predicate: a predicated-off
                // UTCHMMA still costs tensor-pipe time (measured: 0.88 -> 0.98 of the issue
                // peak when the @!P UTCHMMAs are gone, tools/diag_gemm.py).
                if (p.terms == 4) {
#pragma unroll
                  for (int k = 0; k < kBK / 16; k++) {
                    const uint64_t ko = (uint64_t)(k * 2);  // +32 B per 16-wide k step (>>4)
                    const uint32_t first = k > 0 ? 1u : acc0;
                    ptx::mma_f16<CG>(acc_x, d_alo + ko, d_blo + ko, idesc, first);
                    ptx::mma_f16<CG>(acc_x, d_alo + ko, d_bhi + ko, idesc, 1u);
                    ptx::mma_f16<CG>(acc_x, d_ahi + ko, d_blo + ko, idesc, 1u);
                    ptx::mma_f16<CG>(acc_hh, d_ahi + ko, d_bhi + ko, idesc, SEP ? first : 1u);
                  }
                } else {
#pragma unroll
                  for (int k = 0; k < kBK / 16; k++) {
                    const uint64_t ko = (uint64_t)(k * 2);
                    const uint32_t first = k > 0 ? 1u : acc0;
                    ptx::mma_f16<CG>(acc_x, d_alo + ko, d_bhi + ko, idesc, first);
                    ptx::mma_f16<CG>(acc_x, d_ahi + ko, d_blo + ko, idesc, 1u);
                    ptx::mma_f16<CG>(acc_hh, d_ahi + ko, d_bhi + ko, idesc, SEP ? first : 1u);
                  }
                }
                if constexpr (NORM) {
                  // acc += 1 * h_j + 1 * m_j + 1 * l_j = a.b_j - ||b_j||^2 / 2 (reading R22)
                  if (kb == p.num_kb - 1)
                    ptx::mma_tf32<CG>(acc_hh, ptx::sdesc_kmajor_sw32(ptx::smem_u32(ones_tile)),
                                      ptx::sdesc_kmajor_sw32(sa + NP_OFF),
                                      ptx::idesc_tf32_f32(kBM * CG, BN), 1u);
                }
                if (kb == kb0 && ch == 0 && ns == 0) {
                  if (uctr == 0) TL(3);
                  else if (uctr == 1) TL(9);
                }
                if (!(DIAG_NO_TMA && DIAG_MODE(4))) ptx::mma_commit<CG>(&empty[stage]);
                if (!AR && DIAG_MODE(1)) ptx::mma_commit<CG>(a_empty);  // diagnostics only
              }
              __syncwarp();
              if (++stage == STAGES) { stage = 0; phase ^= 1u; }
            }
            if (ptx::elect_one()) {
              ptx::mma_commit<CG>(&acc_full[buf]);
              TL(4);
            }
            __syncwarp();
            chunk_ctr++;
          }
        }
        if constexpr (AR) {  // the resident A tile is free once this unit's MMAs complete
          if (ptx::elect_one()) ptx::mma_commit<CG>(aslot ? a_empty1 : a_empty);
          __syncwarp();
        }
      }
    }
   }
  } else {
    if constexpr (CONV) asm volatile("setmaxnreg.inc.sync.aligned.u32 176;");
    if constexpr (BIGREG) asm volatile("setmaxnreg.inc.sync.aligned.u32 216;");
    // ============================ epilogue ============================
    const int ew = warp - EG::EPI0;
    const int q = warp & 3;         // TMEM lane quarter this warp may access
    const int cgp = ew >> 2;        // column group (0 .. GPQ-1) within the lane quarter
    const uint32_t lane_off = (uint32_t)(q * 32) << 16;
    uint32_t chunk_ctr = 0;
    const int row_in_cta = q * 32 + lane;

    float kd[KN];
    int ki[KN];
    // KREG: the two column groups of a row exchange their sorted key lists once per tile
    // (double-buffered smem slots after the merge scratch, named barrier 5 + q)
    uint32_t xgen = 0;
    uint32_t km_units = 0;  // kMeans: units finished (merge-slot parity)
    float gpend = __int_as_float(0x7fffffff);  // kNN: the row bound loaded at the last exchange
    float gcur = __int_as_float(0x7fffffff);   // kNN: the row bound in use (NaN: none)
    float* const xch = reinterpret_cast<float*>(scratch + kBM * kKnnMerge * 8);
    float best = __int_as_float(0xff800000);
    int besti = 0x7fffffff;

    for (int u = cluster; u < p.num_units; u += nclusters) {
      UnitInfo ui = decode_unit<EPI>(p, u);
      const int64_t row = (int64_t)ui.m_tile * (kBM * CG) + rank * kBM + row_in_cta;
      if constexpr (EPI == EPI_KNN) {
#pragma unroll
        for (int t = 0; t < KN; t++) { kd[t] = __int_as_float(0x7f800000); ki[t] = 0x7fffffff; }
      }
      // kMeans: best = the largest accumulator (= smallest key) so far, key = -2 best
      if constexpr (EPI == EPI_KMEANS) { best = __int_as_float(0xff800000); besti = 0x7fffffff; }

      for (int ns = 0; ns < ui.n_count; ns++) {
        const int col_base = (ui.n_begin + ns) * BN + cgp * COLS;
        if constexpr (EPI == EPI_STORE) {
          float tot[COLS];
          float totx[SEP ? COLS : 1];
#pragma unroll
          for (int j = 0; j < COLS; j++) tot[j] = 0.f;
          if constexpr (SEP) {
#pragma unroll
            for (int j = 0; j < COLS; j++) totx[j] = 0.f;
          }
          const int nch = (ui.kb1 - ui.kb0 + p.kb_per_chunk - 1) / p.kb_per_chunk;
          // split-K: this part's result goes to row block ks of D (the host reduces the parts)
          const int64_t drow0 = p.ksplit > 1 ? (int64_t)ui.ks * p.m_pad : 0;
          for (int ch = 0; ch < nch; ch++) {
            const uint32_t buf = chunk_ctr & 1u;
            const uint32_t use = chunk_ctr >> 1;
            ptx::mbar_wait(&acc_full[buf], use & 1u);
            ptx::tc_fence_after();
            if (ew == 0 && lane == 0) TL(5);
            const uint32_t acc_hh = tmem_base + lane_off + (SEP ? 2 * buf : buf) * BN + cgp * COLS;
            if (!DIAG_NO_EPI)
#pragma unroll
            for (int c = 0; c < COLS / LDW; c++) {
              float v[LDW];
              if constexpr (LDW == 32) ptx::tmem_ld32(acc_hh + c * LDW, v);
              else ptx::tmem_ld16(acc_hh + c * LDW, v);
              ptx::tmem_wait_ld();
#pragma unroll
              for (int i = 0; i < LDW; i++) tot[c * LDW + i] = __fadd_rn(tot[c * LDW + i], v[i]);
              if constexpr (SEP) {
                if constexpr (LDW == 32) ptx::tmem_ld32(acc_hh + BN + c * LDW, v);
                else ptx::tmem_ld16(acc_hh + BN + c * LDW, v);
                ptx::tmem_wait_ld();
#pragma unroll
                for (int i = 0; i < LDW; i++) totx[c * LDW + i] = __fadd_rn(totx[c * LDW + i], v[i]);
              }
            }
            ptx::tc_fence_before();
            __syncwarp();
            if (lane == 0) {
              if constexpr (CG == 1) ptx::mbar_arrive(&acc_empty[buf]);
              else ptx::mbar_arrive_cluster(&acc_empty[buf], 0);
            }
            chunk_ctr++;
          }
          if constexpr (SEP) {
#pragma unroll
            for (int j = 0; j < COLS; j++) tot[j] = __fadd_rn(tot[j], totx[j]);
          }
          if (ew == 0 && lane == 0) TL(12);
          if (ui.fx >= 0) {
            // tail split: this part's sums go to the workspace (coalesced float4 slab per
            // warp); the warp that completes a slab's last part adds the parts in k order
            // (RN, R21 -- the split-K reduce's order) and stores the tile.  No part ever waits.
            constexpr int SLABS = CG * NEPI;
            constexpr int SLAB_F4 = COLS / 4 * 32;
            const int slab = (int)rank * NEPI + ew;
            float4* wsb = reinterpret_cast<float4*>(p.fix_ws) +
                          ((size_t)ui.fx * p.tail_parts * SLABS + slab) * SLAB_F4;
            float4* own = wsb + (size_t)ui.ks * SLABS * SLAB_F4;
#pragma unroll
            for (int j = 0; j < COLS / 4; j++)
              own[j * 32 + lane] = make_float4(tot[4 * j], tot[4 * j + 1], tot[4 * j + 2], tot[4 * j + 3]);
            __threadfence();
            __syncwarp();
            uint32_t old = 0;
            if (lane == 0) old = atomicAdd(p.fix_cnt + (size_t)ui.fx * SLABS + slab, 1u);
            old = __shfl_sync(0xffffffffu, old, 0);
            if (old + 1u != (uint32_t)p.tail_parts) continue;  // another part completes it
            __threadfence();
            // (the own part is read back too: tot need not stay live across the hand-off)
#pragma unroll
            for (int j = 0; j < COLS / 4; j++) {
              float4 a = __ldcg(wsb + j * 32 + lane);
#pragma unroll
              for (int s2 = 1; s2 < 4; s2++) {  // (host: tail_parts <= 4)
                if (s2 < p.tail_parts) {
                  const float4 b = __ldcg(wsb + (size_t)s2 * SLABS * SLAB_F4 + j * 32 + lane);
                  a.x = __fadd_rn(a.x, b.x); a.y = __fadd_rn(a.y, b.y);
                  a.z = __fadd_rn(a.z, b.z); a.w = __fadd_rn(a.w, b.w);
                }
              }
              tot[4 * j] = a.x; tot[4 * j + 1] = a.y; tot[4 * j + 2] = a.z; tot[4 * j + 3] = a.w;
            }
          }
          if constexpr (TS) {
            if (p.tma_store) {
              const uint32_t buf = ts_base + (uint32_t)ew * 4096u;
              const int row0 = (int)drow0 + ui.m_tile * (kBM * CG) + (int)rank * kBM + q * 32;
#pragma unroll
              for (int c = 0; c < COLS / 32; c++) {
                if (lane == 0) ptx::tma_store_wait_read0();  // the previous store read the buffer
                __syncwarp();
#pragma unroll
                for (int k = 0; k < 8; k++)
                  ptx::sts128(buf + lane * 128 + ((k ^ (lane & 7)) << 4), __float_as_uint(tot[c * 32 + 4 * k]),
                              __float_as_uint(tot[c * 32 + 4 * k + 1]), __float_as_uint(tot[c * 32 + 4 * k + 2]),
                              __float_as_uint(tot[c * 32 + 4 * k + 3]));
                ptx::fence_proxy_async_smem();  // generic-proxy writes -> visible to the TMA unit
                __syncwarp();
                if (lane == 0) {  // rows >= M and columns >= N of the box are clipped by TMA
                  ptx::tma_store_2d_u32(&tm_d, buf, col_base + c * 32, row0);
                  ptx::tma_store_commit();
                }
              }
              if (ew == 0 && lane == 0) TL(6);
              continue;
            }
          }
          if (row < p.M) {
            float* drow = p.D + (drow0 + row) * p.ldd;
            const float* crow = p.C ? p.C + row * p.ldc : nullptr;
            if (p.vec_ok && col_base + COLS <= p.N) {
#pragma unroll
              for (int j = 0; j < COLS; j += 4) {
                float4 o = make_float4(tot[j], tot[j + 1], tot[j + 2], tot[j + 3]);
                if (crow) {
                  float4 cv = *reinterpret_cast<const float4*>(crow + col_base + j);
                  o.x = __fadd_rn(o.x, cv.x); o.y = __fadd_rn(o.y, cv.y);
                  o.z = __fadd_rn(o.z, cv.z); o.w = __fadd_rn(o.w, cv.w);
                }
                *reinterpret_cast<float4*>(drow + col_base + j) = o;
              }
            } else {
#pragma unroll
              for (int j = 0; j < COLS; j++) {
                int col = col_base + j;
                if (col < p.N) drow[col] = crow ? __fadd_rn(tot[j], crow[col]) : tot[j];
              }
            }
          }
        } else {
          // kNN / kMeans: one chunk per n-step (host guarantees Kc >= K)
          const uint32_t buf = chunk_ctr & 1u;
          const uint32_t use = chunk_ctr >> 1;
          ptx::mbar_wait(&acc_full[buf], use & 1u);
          ptx::tc_fence_after();
          if (DIAG_MODE(64)) {  // diagnostics only: TMEM reads, no epilogue arithmetic
            const uint32_t a0 = tmem_base + lane_off + buf * BN + cgp * COLS;
#pragma unroll
            for (int c = 0; c < COLS / 32; c++) {
              float v[32];
              ptx::tmem_ld32(a0 + c * 32, v);
              ptx::tmem_wait_ld();
              if (v[c] == 1234.5f) best = v[31];  // keep the loads observable
            }
          }
          if (DIAG_NO_EPI || DIAG_MODE(64)) {  // diagnostics: release untouched
            ptx::tc_fence_before();
            __syncwarp();
            if (lane == 0) {
              if constexpr (CG == 1) ptx::mbar_arrive(&acc_empty[buf]);
              else ptx::mbar_arrive_cluster(&acc_empty[buf], 0);
            }
            chunk_ctr++;
            continue;
          }
          const uint32_t acc_hh = tmem_base + lane_off + (SEP ? 2 * buf : buf) * BN + cgp * COLS;
          if constexpr (KREG) {
            float v[COLS];
#pragma unroll
            for (int c = 0; c < COLS / 32; c++) ptx::tmem_ld32(acc_hh + c * 32, v + c * 32);
            ptx::tmem_wait_ld();
            ptx::tc_fence_before();
            __syncwarp();
            if (lane == 0) {
              if constexpr (CG == 1) ptx::mbar_arrive(&acc_empty[buf]);
              else ptx::mbar_arrive_cluster(&acc_empty[buf], 0);
            }
            // Filter bound u = the 16th smallest key of (own list) U (the partner group's list
            // as published after the previous tile of this unit).  Both lists hold distinct
            // real columns of this row, so at least 16 keys <= u exist and a key > u can never
            // reach the row's final top 16 (a key == u still may, by index: kept).  The union
            // bound cuts the insertions to about those of one list over both column halves.
            float u = kd[KN - 1];
            {
              if (ns > 0) {  // (ns == 0: the last publication belongs to the previous unit's rows)
                const uint32_t pb = ptx::smem_u32(
                    xch + ((((xgen - 1) & 1u) * GPQ + (cgp ^ 1)) * kBM + q * 32 + lane) * KN);
                float b[KN];
#pragma unroll
                for (int t = 0; t < KN / 4; t++) {
                  const float4 w = ptx::lds128f(pb + 16 * t);
                  b[4 * t] = w.x; b[4 * t + 1] = w.y; b[4 * t + 2] = w.z; b[4 * t + 3] = w.w;
                }
                // 16th smallest of two sorted 16-lists: min over splits i of max(A[i-1], B[15-i])
                float m = fminf(b[KN - 1], kd[KN - 1]);
#pragma unroll
                for (int i = 1; i < KN; i++) m = fminf(m, fmaxf(kd[i - 1], b[KN - 1 - i]));
                u = m;
              }
            }
            // Every 8 tiles the bound is also exchanged with the row's other N-slices through
            // global memory (plain loads / stores: any value ever stored is a valid bound, a
            // lost update only loosens it; NaN = none yet).  A slice that starts after
            // another slice of the same rows then skips most of its list warm-up.
            // The unit's first tile waits for the load; later exchanges use the value loaded
            // at the previous one (issued 8 tiles earlier, off the critical path).
            // The bound in use (gcur) applies to every tile; it is refreshed every 8 tiles.
            if (p.row_bound && !DIAG_MODE(512) && row < p.M) {
              if ((ns & 7) == 0) {
                float* gb = p.row_bound + row;
                if (ns == 0) {
                  asm volatile("ld.relaxed.gpu.global.f32 %0, [%1];" : "=f"(gcur) : "l"(gb) : "memory");
                } else {
                  if (!(gpend <= u))
                    asm volatile("st.relaxed.gpu.global.f32 [%0], %1;" ::"l"(gb), "f"(u) : "memory");
                  gcur = fminf(gcur, gpend);
                }
                asm volatile("ld.relaxed.gpu.global.f32 %0, [%1];" : "=f"(gpend) : "l"(gb) : "memory");
              }
              u = fminf(u, gcur);
            }
            // key < own 16th (strict: stream order) and key <= u, in accumulator space
            // (key = -2 v): v > -kd15/2 and v >= -u/2
            const float vt = fmaxf(-0.5f * kd[KN - 1], nextafterf(-0.5f * u, __int_as_float(0xff800000)));
#pragma unroll
            for (int c = 0; c < COLS / 32; c++) {
              float* g = v + c * 32;
              const int c0 = col_base + c * 32;
              if (c0 + 32 > p.N) {  // ragged last tile: columns >= N never win
#pragma unroll
                for (int i = 0; i < 32; i++) g[i] = (c0 + i < p.N) ? g[i] : __int_as_float(0xff800000);
              }
              // v = a.b_j - ||b_j||^2/2, key_j = -2 v (exact).  key < thr <=> v > -thr/2 (the
              // threshold is itself -2 v_k: halving it is exact), so the filter compares the
              // accumulators directly; the group maximum by a tree (depth 5, not a chain of 16).
              float t16[16];
#pragma unroll
              for (int i = 0; i < 16; i++) t16[i] = fmaxf(g[2 * i], g[2 * i + 1]);
#pragma unroll
              for (int w = 8; w >= 1; w >>= 1)
#pragma unroll
                for (int i = 0; i < w; i++) t16[i] = fmaxf(t16[i], t16[i + w]);
              if (__any_sync(0xffffffffu, t16[0] > vt) && !DIAG_MODE(128)) {
                if (DIAG_MODE(256) && lane == 0) atomicAdd(&p.probe[7], 1ull);
                uint32_t cand = 0;
                float vv[32];
#pragma unroll
                for (int i = 0; i < 32; i++) {
                  vv[i] = g[i];
                  cand |= (g[i] > vt) ? (1u << i) : 0u;
                }
                // a thread's columns arrive in increasing index order: strict '<' inside the
                // insertion keeps the lower index first among equal keys
#pragma unroll 1
                while (cand) {
                  const int i = __ffs(cand) - 1;
                  cand &= cand - 1u;
                  topk_insert_stream<KN>(kd, ki, -2.f * vv[i], c0 + i);
                }
              }
            }
            {  // publish this tile's list for the partner group
              const uint32_t ob = ptx::smem_u32(
                  xch + (((xgen & 1u) * GPQ + cgp) * kBM + q * 32 + lane) * KN);
#pragma unroll
              for (int t = 0; t < KN / 4; t++)
                ptx::sts128f(ob + 16 * t, kd[4 * t], kd[4 * t + 1], kd[4 * t + 2], kd[4 * t + 3]);
              // lockstep per tile (a bar.arrive / bar.sync pair could let one warp arrive
              // twice before the other syncs, merging two barrier generations)
              named_bar_sync(5 + q, 64);
              xgen++;
            }
            chunk_ctr++;
            continue;
          }
          // TMEM -> registers software-pipelined: the load of group c+1 is in flight while
          // group c is processed; the accumulator buffer is handed back to the MMA warp as
          // soon as the last group has landed in registers.
          // (with 16 epilogue warps the extra warps hide the latency instead of registers)
          constexpr bool PIPE = (NEPI == 8) && KN == 16;
          float vbuf[PIPE ? 2 : 1][32];
          if (PIPE) ptx::tmem_ld32(acc_hh, vbuf[0]);
#pragma unroll
          for (int c = 0; c < COLS / 32; c++) {
            float* v = vbuf[PIPE ? (c & 1) : 0];
            if (!PIPE) ptx::tmem_ld32(acc_hh + c * 32, v);
            ptx::tmem_wait_ld();
            if constexpr (SEP) {
              float w[32];
              ptx::tmem_ld32(acc_hh + BN + c * 32, w);
              ptx::tmem_wait_ld();
#pragma unroll
              for (int i = 0; i < 32; i++) v[i] = __fadd_rn(v[i], w[i]);
            }
            if (c + 1 < COLS / 32) {
              if (PIPE) ptx::tmem_ld32(acc_hh + (c + 1) * 32, vbuf[(c + 1) & 1]);
            } else {
              ptx::tc_fence_before();
              __syncwarp();
              if (lane == 0) {
                if constexpr (CG == 1) ptx::mbar_arrive(&acc_empty[buf]);
                else ptx::mbar_arrive_cluster(&acc_empty[buf], 0);
              }
            }
            const int c0 = col_base + c * 32;
            // v = a.b_j - ||b_j||^2 / 2 (norm MMA), so key_j = -2 v exactly: min key = max v
            if (c0 + 32 > p.N) {  // ragged last tile: columns >= N never win
#pragma unroll
              for (int i = 0; i < 32; i++) v[i] = (c0 + i < p.N) ? v[i] : __int_as_float(0xff800000);
            }
            if constexpr (EPI == EPI_KNN) {
              float mx = __int_as_float(0xff800000);
#pragma unroll
              for (int i = 0; i < 32; i++) mx = fmaxf(mx, v[i]);
              // candidate test against this row's current k-th key; the (rare) insertions
              // run in a compact loop over the set bits.  A thread's columns arrive in
              // increasing index order, so a strict '<' keeps the lower index first among
              // equal keys.
              const float thr = kd[KN - 1];
              // (debug bit 128, diagnostics only: never take the candidate path)
              if (__any_sync(0xffffffffu, -2.f * mx < thr) && !DIAG_MODE(128)) {
                uint32_t cand = 0;
                float keys[32];
#pragma unroll
                for (int i = 0; i < 32; i++) {
                  keys[i] = -2.f * v[i];
                  cand |= (keys[i] < thr) ? (1u << i) : 0u;
                }
#pragma unroll 1
                while (cand) {
                  const int i = __ffs(cand) - 1;
                  cand &= cand - 1u;
                  topk_insert_stream<KN>(kd, ki, keys[i], c0 + i);
                }
              }
            } else {
              // group max first (3-input FMNMX), the index only when it improves.  (Parking
              // the improving quarter in smem and searching once per unit measured the same.)
              // (a depth-5 tree here, or loading both groups and releasing the accumulator
              // before the search, measured slower than this chain with 16 warps)
              // The search runs for the whole warp whenever one lane improves (nearly every
              // group: the first groups of a row always do), so it is kept short: the half
              // holding the maximum (the lower half on a tie) is selected first, then searched.
              float mxa = __int_as_float(0xff800000), mxb = mxa;
#pragma unroll
              for (int i = 0; i < 16; i++) { mxa = fmaxf(mxa, v[i]); mxb = fmaxf(mxb, v[16 + i]); }
              const float mx = fmaxf(mxa, mxb);
              if (mx > best) {  // strict: an equal key from a later column never wins
                const bool lo = (mxa == mx);
                float w[16];
#pragma unroll
                for (int i = 0; i < 16; i++) w[i] = lo ? v[i] : v[16 + i];
                int idx = 15;
#pragma unroll
                for (int i = 14; i >= 0; i--) idx = (w[i] == mx) ? i : idx;  // lowest index
                best = mx;
                besti = c0 + (lo ? idx : 16 + idx);
              }
            }
          }
          chunk_ctr++;
        }
      }

      // ---- unit end: merge the two column halves of each row, write the unit's result
      if constexpr (EPI == EPI_KNN) {
        // column groups 1..GPQ-1 hand their lists to group 0 one at a time, kKnnMerge entries
        // per round (8 KiB scratch)
        constexpr int KH = kKnnMerge;
        float* sk = reinterpret_cast<float*>(scratch) + (q * 32 + lane) * KH;
        int* si = reinterpret_cast<int*>(scratch + kBM * KH * 4) + (q * 32 + lane) * KH;
#pragma unroll 1
        for (int g = 1; g < GPQ; g++) {
#pragma unroll
          for (int h = 0; h < KN / KH; h++) {
            if (cgp == g) {
#pragma unroll
              for (int t = 0; t < KH; t++) { sk[t] = kd[h * KH + t]; si[t] = ki[h * KH + t]; }
            }
            named_bar_sync(1 + q, 32 * GPQ);
            if (cgp == 0) {
#pragma unroll 1
              for (int t = 0; t < KH; t++) topk_insert<KN>(kd, ki, sk[t], si[t]);
            }
            named_bar_sync(1 + q, 32 * GPQ);
          }
        }
        if (cgp == 0 && row < p.M) {
          const int64_t o = ((int64_t)ui.slice * p.M + row) * p.knn_k;
#pragma unroll
          for (int t = 0; t < KN; t++)
            if (t < p.knn_k) { p.part_key[o + t] = kd[t]; p.part_idx[o + t] = ki[t]; }
        }
      } else if constexpr (EPI == EPI_KMEANS) {
        best = -2.f * best;  // the key (exact): ||c||^2 - 2 x.c
        // merge the GPQ column groups of each row through smem.  The slots alternate with the
        // unit's parity, so only group 0 waits (one barrier per unit): a group writes the
        // same slots again two units later, after the next unit's barrier, which group 0
        // reaches only once it has read these.
        uint8_t* slot = scratch + (km_units & 1u) * (2 * GPQ * kBM * 4);
        km_units++;
        float* sk = reinterpret_cast<float*>(slot);
        int* si = reinterpret_cast<int*>(slot + GPQ * kBM * 4);
        const int r = q * 32 + lane;
        if (cgp > 0) { sk[(cgp - 1) * kBM + r] = best; si[(cgp - 1) * kBM + r] = besti; }
        named_bar_sync(1 + q, 32 * GPQ);
        if (cgp == 0) {
#pragma unroll
          for (int g = 1; g < GPQ; g++) {
            const float ob = sk[(g - 1) * kBM + r];
            const int oi = si[(g - 1) * kBM + r];
            if (ob < best || (ob == best && oi < besti)) { best = ob; besti = oi; }
          }
          if (DIAG_NO_EPI || DIAG_MODE(64)) besti = 0;  // diagnostics: keep the downstream kernels in bounds
          if (row < p.M) { p.assign[row] = besti; p.best_key[row] = best; }
        }
      }
    }
  }

  // ============================ teardown ============================
  if constexpr (TS) {
    // the staging buffers must have been read before the CTA's shared memory goes away; the
    // global writes themselves complete with the grid (a successor -- stream order or its
    // griddepcontrol.wait -- sees them), so the CTA does not wait for them (-0.8 K cycles at
    // the end of every launch, tools/timeline.py)
    if (p.tma_store && warp >= EG::EPI0 && lane == 0) ptx::tma_store_wait_read0();
    if (warp == EG::EPI0 && lane == 0) TL(13);
  }
  __syncwarp();
  ptx::tc_fence_before();
  if constexpr (CG == 2) ptx::cluster_sync(); else __syncthreads();
  if (threadIdx.x == 0) {
    TL(7);
    if (DIAG_MODE(2048) && blockIdx.x == 0) p.probe[8 + 11] = globaltimer_ns();
  }
  if (warp == EG::W_ALLOC) {
    ptx::tc_fence_after();
    ptx::tmem_dealloc<CG>(tmem_base, TMEM_COLS);
  }
  if (blockIdx.x == 0 && threadIdx.x == 0 && !p.pdl_wait) {
    const unsigned long long c1 = clock64(), t1 = globaltimer_ns();
    p.probe[2] = c1;
    p.probe[3] = t1;
    p.probe[4] += c1 - p.probe[0];
    p.probe[5] += t1 - p.probe[1];
    p.probe[6] += 1;
  }
  // a peeled tail launch completes only after the grid it overlapped (its stream successors
  // may overwrite that grid's operands)
  if (p.pdl_wait) asm volatile("griddepcontrol.wait;" ::: "memory");
}

// ------------------------------------------------------------------ launch of one variant
// Dynamic shared memory of a variant (bytes, including the 1 KiB alignment slack).
template <int CG, int BN, int EPI, int STAGES, bool FA, bool AR, bool AS, bool FB, int NEPI, int KN>
constexpr size_t variant_smem() {
  using G = Geo<CG, BN>;
  // kNN: the unit-end merge (kKnnMerge entries per round) + KREG's list exchange (two
  // generations x two column groups x 128 rows of 16-key lists); kMeans: (key, index) of
  // the column groups, two unit parities
  constexpr bool KREG = (EPI == EPI_KNN) && AR && !FA && NEPI == 8 && BN / (NEPI / 4) == 128 && KN == 16;
  constexpr size_t scratch = EPI == EPI_KNN ? kBM * kKnnMerge * 8 + (KREG ? 2 * 2 * kBM * KN * 4 : 0)
                             : EPI == EPI_KMEANS ? 2 * 2 * 4 * kBM * 4 : 0;
  constexpr bool NORM = (EPI != EPI_STORE);  // norm slot per stage + the A' ones tile
  constexpr size_t sb = (AR ? 2 * G::B_BYTES : G::STAGE_BYTES) + (NORM ? G::BNC * 32 : 0);
  constexpr size_t base = 1024 + (size_t)STAGES * sb + (AR ? 4 * G::A_BYTES : 0) + (NORM ? kBM * 32 : 0) +
                          (FB ? 3 * kBM * kBK * 4 + 8 * 6 : 0) + (AS ? 8 * STAGES : 0) +
                          8 * (2 * STAGES + 10) + scratch;
  // TS: one 4 KiB TMA-store staging buffer per epilogue warp, 1 KiB aligned (128-B swizzle)
  constexpr bool TS = (EPI == EPI_STORE) && !FB && ((BN / (NEPI / 4)) % 32 == 0);
  return TS ? ((base + 1023) / 1024) * 1024 + (size_t)NEPI * 4096 : base;
}

template <int CG, int BN, bool SEP, int EPI, int STAGES, bool FA = false, bool AR = false,
          bool AS = false, bool FB = false, int NEPI = 8, int KN = 16>
static int launch_variant(const CUtensorMap* maps, const KParams& kp, int max_clusters,
                          cudaStream_t stream) {
  auto kern = egemm_tc_kernel<CG, BN, SEP, EPI, STAGES, NEPI, FA, AR, AS, FB, KN>;
  constexpr size_t smem = variant_smem<CG, BN, EPI, STAGES, FA, AR, AS, FB, NEPI, KN>();
  static_assert(smem <= 232448, "shared memory of the variant exceeds 227 KiB");
  // the opt-in attributes are per device: one bit per device this variant has launched on
  static std::atomic<unsigned long long> attr_devices{0};
  int dev = 0;
  if (cudaGetDevice(&dev) != cudaSuccess || dev < 0 || dev >= 64) {
    set_last_error("cudaGetDevice failed");
    return 3;
  }
  const unsigned long long bit = 1ull << dev;
  if (!(attr_devices.load(std::memory_order_acquire) & bit)) {
    if (cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem) !=
        cudaSuccess) {
      set_last_error("cudaFuncSetAttribute(smem=%zu) failed", smem);
      return 3;
    }
    if (CG == 2) cudaFuncSetAttribute(kern, cudaFuncAttributeNonPortableClusterSizeAllowed, 0);
    attr_devices.fetch_or(bit, std::memory_order_acq_rel);
  }
  int clusters = num_sms() / CG;
  if (max_clusters > 0 && max_clusters < clusters) clusters = max_clusters;
  if (clusters > kp.num_units) clusters = kp.num_units;
  if (clusters < 1) clusters = 1;
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3((unsigned)(clusters * CG), 1, 1);
  cfg.blockDim = dim3(EpiGeo<NEPI, FA || FB>::THREADS, 1, 1);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = stream;
  cudaLaunchAttribute attr[2];
  attr[0].id = cudaLaunchAttributeClusterDimension;
  attr[0].val.clusterDim.x = CG;
  attr[0].val.clusterDim.y = 1;
  attr[0].val.clusterDim.z = 1;
  attr[1].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[1].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = attr;
  // cluster dims + programmatic stream serialization (see the kernel's setup)
  cfg.numAttrs = (kp.pdl_wait || !knobs().no_pdl) ? 2 : 1;
  cudaError_t e = cudaLaunchKernelEx(&cfg, kern, maps[0], maps[1], maps[2], maps[3], maps[4], kp);
  if (e != cudaSuccess) {
    set_last_error("cudaLaunchKernelEx: %s", cudaGetErrorString(e));
    return 3;
  }
  return 0;
}

// Variant dispatchers (one translation unit each); 2 = no such variant (UNSUPPORTED).
int dispatch_store(const CUtensorMap* maps, const KParams& kp, const TcConfig& cfg, cudaStream_t s);
int dispatch_fused(const CUtensorMap* maps, const KParams& kp, const TcConfig& cfg, cudaStream_t s);
int dispatch_knn(const CUtensorMap* maps, const KParams& kp, const TcConfig& cfg, cudaStream_t s);
int dispatch_kmeans(const CUtensorMap* maps, const KParams& kp, const TcConfig& cfg, cudaStream_t s);

}  // namespace egemm
