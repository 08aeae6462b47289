// gemm_tc.cu -- host side of the tensor-core kernel: TMA descriptors, the kernel parameter
// block, and the dispatch of launch_tc to the variant translation units (tc_store.cu,
// tc_fused.cu, tc_knn.cu, tc_kmeans.cu); the device clock probe read back by the debug calls.
#include "tc_kernel.cuh"

namespace egemm {

// [0..3] last launch, [4..6] running sums, [7] counter, [8..23] phase timeline (EGEMM_DIAG)
__device__ unsigned long long g_clock_probe[24];

static unsigned long long* probe_ptr() {
  void* p = nullptr;
  if (cudaGetSymbolAddress(&p, g_clock_probe) != cudaSuccess) return nullptr;
  return reinterpret_cast<unsigned long long*>(p);
}

// Debug event counter (g_clock_probe[7]).
int read_debug_counter(unsigned long long* value, int reset) {
  if (cudaMemcpyFromSymbol(value, g_clock_probe, sizeof(unsigned long long),
                           7 * sizeof(unsigned long long)) != cudaSuccess)
    return 3;
  if (reset) {
    const unsigned long long z = 0;
    if (cudaMemcpyToSymbol(g_clock_probe, &z, sizeof(z), 7 * sizeof(unsigned long long)) != cudaSuccess)
      return 3;
  }
  return 0;
}

// Phase timeline of CTA 0 (g_clock_probe[8..23], written by EGEMM_DIAG builds).
int read_debug_timeline(unsigned long long* out16, int reset) {
  if (cudaMemcpyFromSymbol(out16, g_clock_probe, 16 * sizeof(unsigned long long),
                           8 * sizeof(unsigned long long)) != cudaSuccess)
    return 3;
  if (reset) {
    const unsigned long long z[16] = {};
    if (cudaMemcpyToSymbol(g_clock_probe, z, sizeof(z), 8 * sizeof(unsigned long long)) != cudaSuccess)
      return 3;
  }
  return 0;
}

// SM cycles / wall ns of CTA 0 over the last launch (debug: effective SM clock).
int read_clock_probe(double* mhz) {
  unsigned long long h[8];
  if (cudaMemcpyFromSymbol(h, g_clock_probe, sizeof(h)) != cudaSuccess) return 3;
  *mhz = (h[3] > h[1]) ? (double)(h[2] - h[0]) * 1e3 / (double)(h[3] - h[1]) : 0.0;
  return 0;
}

// Running sums since the last reset: mean SM clock and CTA-0 cycles per launch.
int read_clock_stats(double* mhz, double* cycles_per_launch, double* launches, int reset) {
  unsigned long long h[8];
  if (cudaMemcpyFromSymbol(h, g_clock_probe, sizeof(h)) != cudaSuccess) return 3;
  *mhz = h[5] ? (double)h[4] * 1e3 / (double)h[5] : 0.0;
  *cycles_per_launch = h[6] ? (double)h[4] / (double)h[6] : 0.0;
  *launches = (double)h[6];
  if (reset) {
    unsigned long long z[3] = {0, 0, 0};
    if (cudaMemcpyToSymbol(g_clock_probe, z, sizeof(z), 4 * sizeof(unsigned long long)) !=
        cudaSuccess)
      return 3;
  }
  return 0;
}

// ------------------------------------------------------------------ host side
static PFN_cuTensorMapEncodeTiled_v12000 get_encode() {
  static PFN_cuTensorMapEncodeTiled_v12000 fn = nullptr;
  static std::once_flag once;
  std::call_once(once, [] {
    cudaDriverEntryPointQueryResult q;
    void* ptr = nullptr;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &ptr, cudaEnableDefault, &q) ==
            cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      fn = reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(ptr);
  });
  return fn;
}

// fp16 [rows x cols] row-major with row stride ld elements; box {64, box_rows}, SW128.
static bool make_tmap_f16(CUtensorMap* m, const void* base, int64_t rows, int64_t cols, int64_t ld,
                          int box_rows) {
  auto enc = get_encode();
  if (!enc) return false;
  cuuint64_t dims[2] = {(cuuint64_t)cols, (cuuint64_t)rows};
  cuuint64_t strides[1] = {(cuuint64_t)(ld * 2)};
  cuuint32_t box[2] = {64u, (cuuint32_t)box_rows};
  cuuint32_t estr[2] = {1u, 1u};
  CUresult r = enc(m, CU_TENSOR_MAP_DATA_TYPE_FLOAT16, 2, const_cast<void*>(base), dims, strides,
                   box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B,
                   CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  return r == CUDA_SUCCESS;
}

// fp32 [rows x cols] row-major (row stride ld elements), box {64, box_rows}, no swizzle:
// only used for L2 prefetches of the fused-split A operand.
static bool make_tmap_f32(CUtensorMap* m, const void* base, int64_t rows, int64_t cols, int64_t ld,
                          int box_rows, int box_cols = 64, bool sw128 = false) {
  auto enc = get_encode();
  if (!enc) return false;
  cuuint64_t dims[2] = {(cuuint64_t)cols, (cuuint64_t)rows};
  cuuint64_t strides[1] = {(cuuint64_t)(ld * 4)};
  cuuint32_t box[2] = {(cuuint32_t)box_cols, (cuuint32_t)box_rows};
  cuuint32_t estr[2] = {1u, 1u};
  CUresult r = enc(m, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, const_cast<void*>(base), dims, strides,
                   box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
                   sw128 ? CU_TENSOR_MAP_SWIZZLE_128B : CU_TENSOR_MAP_SWIZZLE_NONE,
                   CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  return r == CUDA_SUCCESS;
}

static int launch_tc_one(int64_t M, int64_t N, int64_t K, const TcOperands& ops, const TcConfig& cfg,
                         const TcEpilogue& epi, cudaStream_t stream, bool pdl_tail) {
  if (M <= 0 || N <= 0) return 0;
  if (M > INT32_MAX / 2 || N > INT32_MAX / 2) {
    set_last_error("M, N must be < 2^30");
    return 2;
  }
  CUtensorMap maps[5];
  const int bnc = cfg.bn / cfg.cg;
  const bool fa = ops.a_f32 != nullptr && epi.kind == EPI_STORE;
  const bool fb = ops.b_f32 != nullptr && epi.kind == EPI_STORE && !fa;
  if ((!fa && (!make_tmap_f16(&maps[0], ops.a_hi, M, K, ops.lda, kBM) ||
               !make_tmap_f16(&maps[1], ops.a_lo, M, K, ops.lda, kBM))) ||
      (!fb && (!make_tmap_f16(&maps[2], ops.b_hi, N, K, ops.ldb, bnc) ||
               !make_tmap_f16(&maps[3], ops.b_lo, N, K, ops.ldb, bnc))) ||
      (fb && !make_tmap_f32(&maps[2], ops.b_f32, K, N, ops.ldb_f32, kBK, bnc, false))) {
    set_last_error("cuTensorMapEncodeTiled failed (alignment: base 16 B, ld %% 8 == 0)");
    return 2;
  }
  if (fa) {  // A is converted in-kernel: maps[0] = fp32 A for the L2 prefetch (else a placeholder)
    maps[0] = maps[2];
    maps[1] = maps[3];
  }
  if (fb) maps[3] = maps[2];  // fp32 B (row-major K x N) in unswizzled 64 x BNC boxes
  maps[4] = maps[2];  // tm_d placeholder unless the STORE epilogue uses TMA stores (below)
  KParams kp = {};
  kp.K = (int)K;
  kp.fb = fb ? 1 : 0;
  kp.bf16 = cfg.fmt == 1 ? 1 : 0;
  kp.pdl_wait = pdl_tail ? 1 : 0;
  if (kp.bf16 && (fa || fb || epi.kind != EPI_STORE)) {
    set_last_error("bf16 operand parts: pre-split STORE GEMMs only");
    return 2;
  }
  const Knobs& kn = knobs();
  kp.debug_no_tma = kn.dbg_no_tma;
  kp.debug_no_epi = kn.dbg_no_epi;
  kp.debug_mode = kn.dbg_mode;
  kp.probe = probe_ptr();
  if (!kp.probe) {
    set_last_error("cudaGetSymbolAddress(clock probe) failed");
    return 3;
  }
  if (fa) {
    kp.a_f32 = ops.a_f32;
    kp.lda_f32 = ops.lda_f32;
    kp.vec_a = ((ops.lda_f32 % 4) == 0 && ((uintptr_t)ops.a_f32 % 16) == 0) ? 1 : 0;
    kp.a_staged = kn.a_staged && kp.vec_a && cfg.cg == 2 && cfg.bn == 256 && !cfg.sep &&
                  make_tmap_f32(&maps[0], ops.a_f32, M, K, ops.lda_f32, kBM, 32, true);
    // L2 prefetch distance in k-blocks (LDG converters: measured 2 > 4 > 8 > 0 at
    // 65536 x 256 x 1024; staged: EGEMM_AS_PREFETCH)
    kp.a_pf = kp.a_staged ? kn.as_pf : kn.a_pf;
    if (kp.a_pf && !kp.a_staged && !(kp.vec_a && make_tmap_f32(&maps[0], ops.a_f32, M, K, ops.lda_f32, kBM)))
      kp.a_pf = 0;
  }
  kp.M = (int)M;
  kp.N = (int)N;
  kp.num_kb = (int)((K + kBK - 1) / kBK);
  kp.kb_per_chunk = cfg.kc / kBK;
  if (kp.kb_per_chunk < 1) kp.kb_per_chunk = 1;
  {
    const KSplit ks = ksplit_geometry(M, N, K, cfg);
    kp.ksplit = epi.kind == EPI_STORE ? ks.parts : 1;
    kp.kb_per_part = ks.kb_per_part;
    kp.m_pad = (int)ks.m_pad;
    if (kp.ksplit > 1) kp.a_pf = 0;  // (the L2 prefetch follows one k-range per unit)
  }
  kp.terms = cfg.terms;
  kp.m_tiles = (int)((M + kBM * cfg.cg - 1) / (kBM * cfg.cg));
  kp.n_tiles = (int)((N + cfg.bn - 1) / cfg.bn);
  kp.D = epi.D;
  kp.ldd = epi.ldd;
  // k-pacing pays off only over long K (measured: +3-4 % at 8192^3 up to +20-30 % at
  // 16384^3, neutral on short-K shapes): below 64 k-blocks it is skipped with its memset
  kp.sync = (epi.kind == EPI_STORE && cfg.pace && !kn.no_pace && kp.num_kb >= 64) ? epi.sync : nullptr;
  kp.pace_e = kn.pace_e > 0 ? kn.pace_e : kSyncE;
  kp.pace_s = kn.pace_s > 0 ? kn.pace_s : kSyncS;
  if (kp.pace_e < 4) kp.pace_e = 4;  // a pair partner runs <= STAGES k-blocks ahead
  if (kp.pace_s < 2 || kp.pace_s >= kSyncR) kp.pace_s = kSyncS;  // >= 2: no pair deadlock
  kp.band_m = kn.band > 0 ? kn.band : 8;
  if (kp.sync && cudaMemsetAsync(kp.sync, 0, kSyncR * sizeof(uint32_t), stream) != cudaSuccess) {
    set_last_error("memset of the pacing counters failed");
    return 3;
  }
  kp.C = epi.C;
  kp.ldc = epi.ldc;
  // D through TMA stores: STORE without C, 16-B aligned D and row stride (32 x 32 fp32 boxes,
  // 128-B swizzle; the variants with 32-column epilogue groups use it, the others ignore it)
  kp.tma_store = (epi.kind == EPI_STORE && !epi.C && epi.D && (epi.ldd % 4) == 0 &&
                  ((uintptr_t)epi.D % 16) == 0 && !knobs().no_tma_store &&
                  make_tmap_f32(&maps[4], epi.D, cfg.ksplit > 1 ? ksplit_geometry(M, N, K, cfg).parts *
                                ksplit_geometry(M, N, K, cfg).m_pad : M, N, epi.ldd, 32, 32, true))
                     ? 1
                     : 0;
  kp.vec_ok = (epi.D && (epi.ldd % 4 == 0) && ((uintptr_t)epi.D % 16 == 0) &&
               (!epi.C || ((epi.ldc % 4 == 0) && ((uintptr_t)epi.C % 16 == 0))))
                  ? 1
                  : 0;
  kp.bnorm = epi.bnorm;
  kp.knn_k = epi.knn_k;
  kp.row_bound = epi.row_bound;
  kp.part_key = epi.part_key;
  kp.part_idx = epi.part_idx;
  kp.assign = epi.assign;
  kp.best_key = epi.best_key;
  if (epi.kind == EPI_STORE) {
    kp.num_units = kp.m_tiles * kp.n_tiles * kp.ksplit;
    const TailSplit tg = tail_geometry(M, N, K, cfg);
    if (tg.parts > 1 && epi.partial && !pdl_tail) {
      kp.tail_u0 = tg.u0;
      kp.tail_parts = tg.parts;
      kp.tail_kbpp = tg.kbpp;
      kp.fix_ws = epi.partial;
      kp.fix_cnt = reinterpret_cast<uint32_t*>(epi.partial + tg.ws_floats);
      kp.num_units = tg.u0 + tg.tiles * tg.parts;
      if (cudaMemsetAsync(kp.fix_cnt, 0, tg.cnt_words * sizeof(uint32_t), stream) != cudaSuccess) {
        set_last_error("memset of the tail-split counters failed");
        return 3;
      }
    }
    return (fa || fb) ? dispatch_fused(maps, kp, cfg, stream) : dispatch_store(maps, kp, cfg, stream);
  }
  if (kp.num_kb > kp.kb_per_chunk) {
    set_last_error("fused kNN/kMeans epilogues need Kc >= K");
    return 2;
  }
  if (epi.kind == EPI_KNN) {
    kp.n_slices = epi.n_slices;
    kp.tiles_per_slice = (kp.n_tiles + epi.n_slices - 1) / epi.n_slices;
    kp.num_units = kp.m_tiles * epi.n_slices;
    return dispatch_knn(maps, kp, cfg, stream);
  }
  kp.num_units = kp.m_tiles;
  return dispatch_kmeans(maps, kp, cfg, stream);
}

// Tail peel (STORE, one n-tile of CTA-pair tiles): when the persistent grid's last wave of
// 256-row units would be at most 60 % full, the rows of that wave go to a second launch of
// 128 x 128 single-CTA tiles (the same per-element arithmetic: same Kc, terms, accumulator
// mode, so the results are bitwise those of one launch).  The second launch is a
// programmatic dependent launch: its CTAs start on the SMs the main grid frees as it
// drains, instead of the freed SMs idling until the main grid's slowest cluster ends; it
// waits for the main grid before it completes, so stream order is kept for later work.
KSplit ksplit_geometry(int64_t M, int64_t N, int64_t K, const TcConfig& cfg) {
  KSplit g = {1, (int)((K + kBK - 1) / kBK), M, N};
  const int num_kb = (int)((K + kBK - 1) / kBK);
  if (cfg.ksplit > 1 && num_kb > 1) {
    const int q = (num_kb + cfg.ksplit - 1) / cfg.ksplit;
    g.parts = (num_kb + q - 1) / q;
    g.kb_per_part = q;
    const int64_t th = (int64_t)kBM * cfg.cg;
    g.m_pad = (M + th - 1) / th * th;
    g.ld = (N + 3) / 4 * 4;
  }
  return g;
}

size_t ksplit_ws_bytes(int64_t M, int64_t N, int64_t K, const TcConfig& cfg) {
  const KSplit g = ksplit_geometry(M, N, K, cfg);
  return g.parts > 1 ? (size_t)g.parts * (size_t)g.m_pad * (size_t)g.ld * sizeof(float) : 0;
}

// The persistent grid runs `clusters` units at a time; when the last wave holds rem <= half
// of them, its tiles' k-range is cut into parts = min(4, clusters / rem) parts run side by
// side, so the last wave takes ~1/parts of a wave instead of a whole one.
TailSplit tail_geometry(int64_t M, int64_t N, int64_t K, const TcConfig& cfg) {
  TailSplit t = {0, 0, 0, 0, 0, 0};
  if (cfg.tsplit <= 0 || cfg.ksplit > 1 || cfg.peel > 0 || M <= 0 || N <= 0 || K <= 0) return t;
  const int num_kb = (int)((K + kBK - 1) / kBK);
  if (num_kb < 4) return t;
  int clusters = num_sms() / cfg.cg;
  if (cfg.max_clusters > 0 && cfg.max_clusters < clusters) clusters = cfg.max_clusters;
  const int64_t th = (int64_t)kBM * cfg.cg;
  const int64_t tiles = ((M + th - 1) / th) * ((N + cfg.bn - 1) / cfg.bn);
  // (a single partly filled wave -- tiles < clusters -- is its own last wave: all of its tiles
  // become k-parts, e.g. 1024^3 at 256 x 128 pair tiles: 32 tiles on 74 clusters)
  if (clusters < 2) return t;
  const int64_t rem = tiles % clusters;
  if (rem == 0 || 2 * rem > clusters) return t;
  int parts = (int)(clusters / rem);
  if (parts > 4) parts = 4;
  if (parts > num_kb / 2) parts = num_kb / 2;
  const int kbpp = (num_kb + parts - 1) / parts;
  parts = (num_kb + kbpp - 1) / kbpp;  // no empty part
  if (parts < 2) return t;
  t.u0 = (int)(tiles - rem);
  t.tiles = (int)rem;
  t.parts = parts;
  t.kbpp = kbpp;
  t.ws_floats = (size_t)rem * parts * (size_t)th * cfg.bn;
  t.cnt_words = (size_t)rem * cfg.cg * 16;  // one counter per epilogue warp (<= 16 per CTA)
  return t;
}

size_t parts_ws_bytes(int64_t M, int64_t N, int64_t K, const TcConfig& cfg) {
  if (const size_t b = ksplit_ws_bytes(M, N, K, cfg)) return b;
  const TailSplit t = tail_geometry(M, N, K, cfg);
  return t.parts > 1 ? t.ws_floats * sizeof(float) + t.cnt_words * sizeof(uint32_t) : 0;
}

// D = fold over the parts in k order (RN) of the split-K part results (+ C last): the
// promotion reading's combination of R21's k-parts.
__global__ void __launch_bounds__(256) ksplit_reduce_kernel(const float* __restrict__ part, int parts,
                                                            int64_t M, int64_t N, int64_t m_pad,
                                                            int64_t ldp, const float* __restrict__ C,
                                                            int64_t ldc, float* __restrict__ D,
                                                            int64_t ldd) {
  const int64_t total = M * N;
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < total; e += stride) {
    const int64_t i = e / N, j = e - i * N;
    float v = part[i * ldp + j];
    for (int s = 1; s < parts; s++) v = __fadd_rn(v, part[((int64_t)s * m_pad + i) * ldp + j]);
    if (C) v = __fadd_rn(v, C[i * ldc + j]);
    D[i * ldd + j] = v;
  }
}

int launch_tc(int64_t M, int64_t N, int64_t K, const TcOperands& ops, const TcConfig& cfg,
              const TcEpilogue& epi, cudaStream_t stream) {
  const bool fb = ops.b_f32 != nullptr && ops.a_f32 == nullptr;
  if (epi.kind == EPI_STORE && cfg.ksplit > 1) {
    const KSplit g = ksplit_geometry(M, N, K, cfg);
    if (g.parts > 1) {
      if (!epi.partial) {
        set_last_error("split-K: no parts buffer (workspace)");
        return 2;
      }
      TcEpilogue e2 = epi;
      e2.D = epi.partial;
      e2.ldd = g.ld;
      e2.C = nullptr;
      int r = launch_tc_one(M, N, K, ops, cfg, e2, stream, false);
      if (r) return r;
      int64_t blocks = (M * N + 255) / 256;
      const int64_t cap = (int64_t)num_sms() * 8;
      if (blocks > cap) blocks = cap;
      ksplit_reduce_kernel<<<(unsigned)blocks, 256, 0, stream>>>(epi.partial, g.parts, M, N, g.m_pad, g.ld,
                                                                 epi.C, epi.ldc, epi.D, epi.ldd);
      return cudaGetLastError() == cudaSuccess ? 0 : 3;
    }
  }
  if (epi.kind == EPI_STORE && cfg.peel > 0 && cfg.cg == 2 && (cfg.bn == 256 || cfg.bn == 224) &&
      !fb && N <= cfg.bn && M > 0) {
    int clusters = num_sms() / 2;
    if (cfg.max_clusters > 0 && cfg.max_clusters < clusters) clusters = cfg.max_clusters;
    const int64_t units = (M + 255) / 256;
    const int64_t full = units / (clusters > 0 ? clusters : 1), rem = units % (clusters > 0 ? clusters : 1);
    if (clusters > 0 && full >= 1 && rem > 0 && rem * 10 <= (int64_t)clusters * 6) {
      const int64_t M1 = full * clusters * 256;
      int r = launch_tc_one(M1, N, K, ops, cfg, epi, stream, false);
      if (r) return r;
      TcOperands t = ops;
      if (ops.a_f32) t.a_f32 = ops.a_f32 + M1 * ops.lda_f32;
      if (ops.a_hi) {
        t.a_hi = ops.a_hi + M1 * ops.lda;
        t.a_lo = ops.a_lo + M1 * ops.lda;
      }
      TcConfig c2 = cfg;
      c2.cg = 1;
      c2.bn = 128;
      c2.stages = 0;
      c2.max_clusters = 0;
      TcEpilogue e2 = epi;
      e2.D = epi.D + M1 * epi.ldd;
      if (epi.C) e2.C = epi.C + M1 * epi.ldc;
      e2.sync = nullptr;
      return launch_tc_one(M - M1, N, K, t, c2, e2, stream, true);
    }
  }
  return launch_tc_one(M, N, K, ops, cfg, epi, stream, false);
}

}  // namespace egemm
