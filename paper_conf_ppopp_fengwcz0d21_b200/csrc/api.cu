// api.cu -- the extern "C" boundary of libegemm.so (declared in include/egemm.h):
// argument validation, tile/term/promotion selection (the tuning table),
// workspace carving, and the launch sequence of each call.  No allocation, no sync.
#include <cuda_runtime.h>
#include <cstdarg>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <mutex>
#include <thread>
#include <nvtx3/nvToolsExt.h>
#include "../../include/egemm.h"
#include "egemm_internal.h"

namespace egemm {

static thread_local char g_err[512] = "";
void set_last_error(const char* fmt, ...) {
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(g_err, sizeof(g_err), fmt, ap);
  va_end(ap);
}

int num_sms() {
  int dev = 0, n = 0;
  if (cudaGetDevice(&dev) != cudaSuccess) return 0;
  if (cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev) != cudaSuccess) return 0;
  return n;
}

static bool device_ok() {
  int dev = 0, major = 0, minor = 0;
  if (cudaGetDevice(&dev) != cudaSuccess) return false;
  cudaDeviceGetAttribute(&major, cudaDevAttrComputeCapabilityMajor, dev);
  cudaDeviceGetAttribute(&minor, cudaDevAttrComputeCapabilityMinor, dev);
  return major == 10 && minor == 0;
}

// ------------------------------------------------------------------ environment knobs
static int env_int(const char* name, int dflt) {
  const char* v = getenv(name);
  return (v && *v) ? atoi(v) : dflt;
}

const Knobs& knobs() {
  static Knobs k;
  static std::once_flag once;
  std::call_once(once, [] {
    k.pace_e = env_int("EGEMM_PACE_E", 0);
    k.pace_s = env_int("EGEMM_PACE_S", 0);
    k.no_pace = env_int("EGEMM_NO_PACE", 0) == 1;
    k.band = env_int("EGEMM_BAND", 0);
    k.a_pf = env_int("EGEMM_A_PREFETCH", 2);
    if (k.a_pf < 0) k.a_pf = 0;
    k.a_staged = env_int("EGEMM_A_STAGED", 1);
    k.as_pf = env_int("EGEMM_AS_PREFETCH", 0);
    if (k.as_pf < 0) k.as_pf = 0;
    k.host_chunk = env_int("EGEMM_HOST_CHUNK", 0);
    k.no_tma_store = env_int("EGEMM_NO_TMA_STORE", 0) == 1;
    k.no_pdl = env_int("EGEMM_NO_PDL", 0) == 1;
#if EGEMM_DIAG
    k.dbg_no_tma = env_int("EGEMM_DEBUG_NO_TMA", 0) == 1;
    k.dbg_no_epi = env_int("EGEMM_DEBUG_NO_EPI", 0) == 1;
    k.dbg_mode = env_int("EGEMM_DEBUG_MODE", 0);
#else
    k.dbg_no_tma = k.dbg_no_epi = k.dbg_mode = 0;
#endif
  });
  return k;
}

// ------------------------------------------------------------------ tuning table
// Measured choices (tools/tune_sweep.py -> tune_table.json): key = (op,
// M/N/K buckets), value = the launch configuration.  The thread-local override
// (egemm_set_config / egemm_set_config_ex) replaces what it sets.
static thread_local egemm_config_t g_override = {};
static thread_local bool g_override_on = false;

static bool fused_a_supported(const TcConfig& c) {
  return (c.cg == 2 && c.bn == 256 && !c.sep) || (c.cg == 2 && c.bn == 128) ||
         (c.cg == 1 && c.bn == 128 && c.sep);
}

static bool valid_config(int cg, int bn, int sep) {
  return (cg == 2 && bn == 256 && sep == 0) || (cg == 1 && bn == 128) ||
         (cg == 2 && bn == 128) || (cg == 2 && bn == 224 && sep == 0);
}

static bool fused_b_supported(const TcConfig& c) {
  return c.cg == 2 && (c.bn == 256 || c.bn == 224) && !c.sep;
}

// b_f32: a STORE GEMM whose B is fp32 (split inside the call): the table's "gemm_b32" rows
// (which may pick the fused-B kernel) first, then the "gemm" rows.  terms: the call's
// argument (0 = the table's choice).
static TcConfig choose_config(int epi_kind, int64_t M, int64_t N, int64_t K, int terms,
                              bool b_f32 = false) {
  TcConfig c = {};
  c.terms = 3;
  c.max_clusters = 0;
  c.cg = 2;  // default: CTA pair, 256 x 256 tiles, single accumulator in ping-pong
  c.bn = 256;
  c.sep = 0;
  c.kc = 64;  // promotion every 64 k: the most accurate single-accumulator setting
  c.ares = -1;
  c.pace = 1;
  c.peel = 0;  // measured slower on configs[2] (profiles/r02_skinny_peel.txt): table / override only
  c.tsplit = 0;  // tail split: fewer cycles but no faster under the power cap (profiles/r02_tail_split_ab.json)
  if (epi_kind == EPI_STORE && M <= 128) { c.cg = 1; c.bn = 128; c.sep = 1; }
  {
    TuneEntry t;
    bool hit = epi_kind == EPI_STORE && b_f32 && tune_lookup(kOpGemmB32, M, N, K, &t) &&
               valid_config(t.cg, t.bn, t.sep);
    if (!hit) hit = tune_lookup(epi_kind, M, N, K, &t) && valid_config(t.cg, t.bn, t.sep);
    if (hit) {
      c.cg = t.cg;
      c.bn = t.bn;
      c.sep = t.sep;
      c.fa = t.fa;
      if (t.kc > 0) c.kc = t.kc;
      if (t.terms == 3 || t.terms == 4) c.terms = t.terms;
      c.stages = t.stages;
      c.nslices = t.nslices;
      c.nepi = t.nepi;
      if (t.ares >= 0) c.ares = t.ares;
      if (t.peel >= 0) c.peel = t.peel;
      if (t.ksplit > 1) c.ksplit = t.ksplit;
      if (t.tsplit >= 0) c.tsplit = t.tsplit;
    }
  }
  if (terms == 3 || terms == 4) c.terms = terms;  // the call's explicit term count wins
  if (epi_kind != EPI_STORE) c.kc = (int)(((K + 63) / 64) * 64);
  if (g_override_on) {  // thread-local API override
    const egemm_config_t& o = g_override;
    if (o.cg) {
      c.cg = o.cg;
      c.bn = o.bn;
      c.sep = o.sep;
      c.fa = 0;  // an explicit tile override measures the pre-split path unless `fused` says
      c.stages = 0;
      c.tsplit = 0;  // ... and no tail split / split-K unless `tail_split` / `ksplit` say
      c.ksplit = 0;
    }
    if (o.kc && epi_kind == EPI_STORE) c.kc = o.kc;
    if (o.fused >= 0) c.fa = o.fused;
    if (o.stages) c.stages = o.stages;
    if (o.terms == 3 || o.terms == 4) c.terms = o.terms;
    if (o.n_slices) c.nslices = o.n_slices;
    if (o.epi_warps) c.nepi = o.epi_warps;
    if (o.a_resident >= 0) c.ares = o.a_resident;
    if (o.pace >= 0) c.pace = o.pace;
    if (o.max_clusters) c.max_clusters = o.max_clusters;
    if (o.tail_peel >= 0) c.peel = o.tail_peel;
    if (o.ksplit) c.ksplit = o.ksplit;
    if (o.tail_split >= 0) c.tsplit = o.tail_split;
    if (o.operand_format == 1 && epi_kind == EPI_STORE) {
      c.fmt = 1;
      c.fa = 0;  // the fused converters produce fp16 parts only
    }
  }
  if (c.kc < 64) c.kc = 64;
  c.kc = (c.kc / 64) * 64;
  if (epi_kind != EPI_STORE) {  // kNN / kMeans: one accumulator (the norm MMA adds into it)
    c.ksplit = 0;
    c.sep = 0;
    c.terms = 3;
    if (!((c.cg == 2 && c.bn == 256) || (c.cg == 1 && c.bn == 128))) { c.cg = 2; c.bn = 256; }
  }
  return c;
}

static size_t align256(size_t x) { return (x + 255) & ~size_t(255); }
static int64_t ldk_of(int64_t K) { return ((K + 7) / 8) * 8; }

struct Carver {
  char* base;
  size_t off = 0;
  template <class T>
  T* take(size_t count) {
    T* p = base ? reinterpret_cast<T*>(base + off) : nullptr;
    off += align256(count * sizeof(T));
    return p;
  }
};

// Make K-major hi/lo of an operand: pre-split pointers if given, else split into ws.
// rows x K logical (K-major).  f32 layout: trans==0 -> rows x K (ld), trans==1 -> K x rows.
static int stage_operand(const egemm_operand_t& op, int64_t rows, int64_t K, Carver& cv,
                         const uint16_t** hi, const uint16_t** lo, int64_t* ld,
                         cudaStream_t s, int mode = 0, bool pdl = false) {
  if (op.hi && op.lo) {
    *hi = op.hi;
    *lo = op.lo;
    *ld = op.ld_split;
    return 0;
  }
  const int64_t ldk = ldk_of(K);
  uint16_t* h = cv.take<uint16_t>((size_t)(rows * ldk));
  uint16_t* l = cv.take<uint16_t>((size_t)(rows * ldk));
  int r = op.trans ? launch_split(op.f32, K, rows, op.ld, h, l, ldk, 1, nullptr, s, mode, pdl && !knobs().no_pdl)
                   : launch_split(op.f32, rows, K, op.ld, h, l, ldk, 0, nullptr, s, mode, pdl && !knobs().no_pdl);
  if (r) {
    set_last_error("split launch failed");
    return EGEMM_ERR_CUDA;
  }
  *hi = h;
  *lo = l;
  *ld = ldk;
  return 0;
}

static int check_operand(const egemm_operand_t& op, int64_t rows, int64_t K, bool is_b,
                         const char* name) {
  bool pre = op.hi && op.lo;
  if ((op.hi == nullptr) != (op.lo == nullptr)) {
    set_last_error("%s: give both hi and lo or neither", name);
    return EGEMM_ERR_INVALID_ARG;
  }
  if (pre) {
    if (op.ld_split < K || (op.ld_split % 8) != 0 || ((uintptr_t)op.hi % 16) ||
        ((uintptr_t)op.lo % 16)) {
      set_last_error("%s: pre-split ld_split must be >= K, a multiple of 8, 16-B aligned", name);
      return op.ld_split < K ? EGEMM_ERR_INVALID_ARG : EGEMM_ERR_UNSUPPORTED;
    }
    return 0;
  }
  if (!op.f32) {
    set_last_error("%s: NULL data", name);
    return EGEMM_ERR_INVALID_ARG;
  }
  // logical rows x K; stored (trans xor is_b) ? K x rows : rows x K
  const bool k_outer = is_b ? !op.trans : op.trans;
  const int64_t need = k_outer ? rows : K;
  if (op.ld < need) {
    set_last_error("%s: ld=%lld < %lld", name, (long long)op.ld, (long long)need);
    return EGEMM_ERR_INVALID_ARG;
  }
  return 0;
}

}  // namespace egemm

using namespace egemm;

// NVTX range around each public compute call (header-only NVTX 3: a no-op unless a
// profiler such as Nsight Systems is attached), so timelines show the C-ABI calls by name.
namespace {
struct NvtxRange {
  explicit NvtxRange(const char* name) { nvtxRangePushA(name); }
  ~NvtxRange() { nvtxRangePop(); }
};
}  // namespace

extern "C" {

const char* egemm_status_string(int s) {
  switch (s) {
    case EGEMM_OK: return "EGEMM_OK";
    case EGEMM_ERR_INVALID_ARG: return "EGEMM_ERR_INVALID_ARG";
    case EGEMM_ERR_UNSUPPORTED: return "EGEMM_ERR_UNSUPPORTED";
    case EGEMM_ERR_CUDA: return "EGEMM_ERR_CUDA";
    case EGEMM_ERR_WORKSPACE: return "EGEMM_ERR_WORKSPACE";
  }
  return "EGEMM_ERR_UNKNOWN";
}

const char* egemm_last_error(void) { return g_err; }
int egemm_version(void) { return 100; }
int egemm_num_sms(void) { return num_sms(); }

const char* egemm_tune_table(int* entries) {
  if (entries) *entries = tune_table_size();
  return tune_table_path();
}

static int knn_slices(int64_t nq, int64_t nx, int cg, int bn);

static void to_public(const TcConfig& c, int op, egemm_config_t* o) {
  const bool b32 = op == kOpGemmB32;
  const bool store = op == EPI_STORE || b32;
  o->cg = c.cg;
  o->bn = c.bn;
  o->sep = c.sep;
  o->kc = c.kc;
  o->stages = c.stages;
  const int a = (store && (c.fa & 1) && fused_a_supported(c)) ? 1 : 0;
  o->fused = a ? 1 : (b32 && (c.fa & 2) && fused_b_supported(c)) ? 2 : 0;
  o->terms = c.terms;
  o->n_slices = c.nslices;
  o->epi_warps = op == EPI_KMEANS ? (c.nepi == 8 ? 8 : 16) : 0;
  o->a_resident = c.ares;
  o->pace = c.pace;
  o->max_clusters = c.max_clusters;
  o->operand_format = c.fmt;
  o->tail_peel = c.peel;
  o->ksplit = c.ksplit > 1 ? c.ksplit : 1;
  o->tail_split = c.tsplit > 0 ? 1 : 0;
}

int egemm_query_config(int op, int64_t M, int64_t N, int64_t K, int* cg, int* bn, int* sep,
                       int* kc, int* fused_a) {
  if (op < 0 || op > 3 || !cg || !bn || !sep || !kc) return EGEMM_ERR_INVALID_ARG;
  egemm_config_t o;
  egemm_query_config_ex(op, M, N, K, &o);
  *cg = o.cg;
  *bn = o.bn;
  *sep = o.sep;
  *kc = o.kc;
  if (fused_a) *fused_a = o.fused;
  return EGEMM_OK;
}

int egemm_query_config_ex(int op, int64_t M, int64_t N, int64_t K, egemm_config_t* out) {
  if (op < 0 || op > 3 || !out) return EGEMM_ERR_INVALID_ARG;
  const bool b32 = op == kOpGemmB32;
  TcConfig c = choose_config(b32 ? EPI_STORE : op, M, N, K, 0, b32);
  if (op == EPI_KNN && c.nslices <= 0) c.nslices = knn_slices(M, N, c.cg, c.bn);
  to_public(c, op, out);
  return EGEMM_OK;
}

int egemm_debug_last_clock(double* mhz) {
  if (!mhz) return EGEMM_ERR_INVALID_ARG;
  return read_clock_probe(mhz) ? EGEMM_ERR_CUDA : EGEMM_OK;
}

int egemm_tc_probe(int kind, int N, int K, const void* A, const void* B, const float* C,
                   float* D, void* stream) {
  if (kind < 0 || kind > 2 || N < 16 || N > 256 || (N % 16) != 0 || K < 1 ||
      K > (kind == 2 ? 128 : 256)) {
    set_last_error("egemm_tc_probe: kind %d, N %d, K %d out of range", kind, N, K);
    return EGEMM_ERR_INVALID_ARG;
  }
  if (!A || !B || !D) {
    set_last_error("egemm_tc_probe: NULL data");
    return EGEMM_ERR_INVALID_ARG;
  }
  if (!device_ok()) {
    set_last_error("no sm_100 device");
    return EGEMM_ERR_CUDA;
  }
  if (launch_tc_probe(kind, N, K, A, B, C, D, (cudaStream_t)stream)) {
    set_last_error("egemm_tc_probe: launch failed");
    return EGEMM_ERR_CUDA;
  }
  return EGEMM_OK;
}

int egemm_debug_clock_stats(double* mhz, double* cycles_per_launch, double* launches, int reset) {
  if (!mhz || !cycles_per_launch || !launches) return EGEMM_ERR_INVALID_ARG;
  return read_clock_stats(mhz, cycles_per_launch, launches, reset) ? EGEMM_ERR_CUDA : EGEMM_OK;
}

int egemm_debug_counter(unsigned long long* value, int reset) {
  if (!value) return EGEMM_ERR_INVALID_ARG;
  return read_debug_counter(value, reset) ? EGEMM_ERR_CUDA : EGEMM_OK;
}

int egemm_debug_timeline(unsigned long long* out, int reset) {
  if (!out) return EGEMM_ERR_INVALID_ARG;
  return read_debug_timeline(out, reset) ? EGEMM_ERR_CUDA : EGEMM_OK;
}

int egemm_set_config(int cg, int bn, int sep, int kc) {
  if (cg == 0 && bn == 0 && sep == 0 && kc == 0) return egemm_set_config_ex(nullptr);
  egemm_config_t o = {};
  o.cg = cg;
  o.bn = bn;
  o.sep = sep;
  o.kc = kc;
  o.fused = -1;
  o.a_resident = -1;
  o.pace = -1;
  o.tail_peel = -1;
  o.tail_split = -1;
  return egemm_set_config_ex(&o);
}

int egemm_set_config_ex(const egemm_config_t* cfg) {
  if (!cfg) {
    g_override = egemm_config_t{};
    g_override_on = false;
    return EGEMM_OK;
  }
  const egemm_config_t& o = *cfg;
  if ((o.cg && !valid_config(o.cg, o.bn, o.sep)) || o.kc < 0 || (o.kc % 64) != 0 ||
      o.fused < -1 || o.fused > 2 || o.stages < 0 || o.stages > 4 ||
      !(o.terms == 0 || o.terms == 3 || o.terms == 4) || o.n_slices < 0 || o.n_slices > 16 ||
      !(o.epi_warps == 0 || o.epi_warps == 8 || o.epi_warps == 16) || o.a_resident < -1 ||
      o.a_resident > 1 || o.pace < -1 || o.pace > 1 || o.max_clusters < 0 ||
      o.operand_format < 0 || o.operand_format > 1 || o.tail_peel < -1 || o.tail_peel > 1 ||
      o.ksplit < 0 || o.ksplit > 16 || o.tail_split < -1 || o.tail_split > 1) {
    set_last_error("unsupported config cg=%d bn=%d sep=%d kc=%d fused=%d stages=%d terms=%d "
                   "n_slices=%d epi_warps=%d", o.cg, o.bn, o.sep, o.kc, o.fused, o.stages, o.terms,
                   o.n_slices, o.epi_warps);
    return EGEMM_ERR_UNSUPPORTED;
  }
  g_override = o;
  g_override_on = true;
  return EGEMM_OK;
}

static int split_entry(const float* x, int64_t rows, int64_t cols, int64_t ldx, uint16_t* hi,
                       uint16_t* lo, int64_t ldo, int transpose, uint32_t* range_flags,
                       void* stream, int mode);

int egemm_split(const float* x, int64_t rows, int64_t cols, int64_t ldx, uint16_t* hi,
                uint16_t* lo, int64_t ldo, int transpose, uint32_t* range_flags, void* stream) {
  NvtxRange nvtx_range("egemm_split");
  return split_entry(x, rows, cols, ldx, hi, lo, ldo, transpose, range_flags, stream, 0);
}

int egemm_split_trunc(const float* x, int64_t rows, int64_t cols, int64_t ldx, uint16_t* hi,
                      uint16_t* lo, int64_t ldo, int transpose, uint32_t* range_flags,
                      void* stream) {
  NvtxRange nvtx_range("egemm_split_trunc");
  return split_entry(x, rows, cols, ldx, hi, lo, ldo, transpose, range_flags, stream, 1);
}

int egemm_split_bf16(const float* x, int64_t rows, int64_t cols, int64_t ldx, uint16_t* hi,
                     uint16_t* lo, int64_t ldo, int transpose, void* stream) {
  NvtxRange nvtx_range("egemm_split_bf16");
  return split_entry(x, rows, cols, ldx, hi, lo, ldo, transpose, nullptr, stream, 2);
}

static int split_entry(const float* x, int64_t rows, int64_t cols, int64_t ldx, uint16_t* hi,
                       uint16_t* lo, int64_t ldo, int transpose, uint32_t* range_flags,
                       void* stream, int mode) {
  if (rows < 0 || cols < 0) {
    set_last_error("negative size");
    return EGEMM_ERR_INVALID_ARG;
  }
  if (rows == 0 || cols == 0) return EGEMM_OK;
  if (!x || !hi || !lo) {
    set_last_error("NULL pointer");
    return EGEMM_ERR_INVALID_ARG;
  }
  if (ldx < cols || ldo < (transpose ? rows : cols)) {
    set_last_error("ld too small");
    return EGEMM_ERR_INVALID_ARG;
  }
  if (!device_ok()) {
    set_last_error("no sm_100 device");
    return EGEMM_ERR_CUDA;
  }
  if (launch_split(x, rows, cols, ldx, hi, lo, ldo, transpose, range_flags, (cudaStream_t)stream,
                   mode)) {
    set_last_error("split launch: %s", cudaGetErrorString(cudaGetLastError()));
    return EGEMM_ERR_CUDA;
  }
  return EGEMM_OK;
}

// Bytes the operand splits need; the full workspace size adds kPaceBytes for the k-pacing
// counters (optional: egemm_gemm runs unpaced when the workspace has no room for them).
static constexpr size_t kPaceBytes = 256;
static size_t gemm_operand_ws(int64_t M, int64_t N, int64_t K, int a_presplit, int b_presplit) {
  if (M <= 0 || N <= 0 || K <= 0) return 0;
  Carver cv{nullptr};
  const int64_t ldk = ldk_of(K);
  if (!a_presplit) { cv.take<uint16_t>((size_t)(M * ldk)); cv.take<uint16_t>((size_t)(M * ldk)); }
  if (!b_presplit) { cv.take<uint16_t>((size_t)(N * ldk)); cv.take<uint16_t>((size_t)(N * ldk)); }
  return cv.off;
}

size_t egemm_gemm_workspace_size(int64_t M, int64_t N, int64_t K, int a_presplit,
                                 int b_presplit) {
  if (M <= 0 || N <= 0 || K <= 0) return 0;
  // (+ the split-K parts buffer when the table / this thread's override picks split-K)
  const TcConfig cfg = choose_config(EPI_STORE, M, N, K, 0, !b_presplit);
  return gemm_operand_ws(M, N, K, a_presplit, b_presplit) +
         ((parts_ws_bytes(M, N, K, cfg) + 255) & ~size_t(255)) + kPaceBytes;
}

int egemm_gemm(int64_t M, int64_t N, int64_t K, egemm_operand_t A, egemm_operand_t B,
               const float* C, int64_t ldc, float* D, int64_t ldd, int terms, void* workspace,
               size_t workspace_bytes, void* stream) {
  NvtxRange nvtx_range("egemm_gemm");
  cudaStream_t s = (cudaStream_t)stream;
  if (M < 0 || N < 0 || K < 0) {
    set_last_error("negative size");
    return EGEMM_ERR_INVALID_ARG;
  }
  if (terms == 0) terms = 3;
  if (terms != 3 && terms != 4) {
    set_last_error("terms must be 0, 3 or 4");
    return EGEMM_ERR_INVALID_ARG;
  }
  if (M == 0 || N == 0) return EGEMM_OK;
  if (!D || ldd < N || (C && ldc < N)) {
    set_last_error("D NULL or ldd/ldc < N");
    return EGEMM_ERR_INVALID_ARG;
  }
  if (!device_ok()) {
    set_last_error("no sm_100 device");
    return EGEMM_ERR_CUDA;
  }
  if (K == 0) return launch_fill_c(M, N, C, ldc, D, ldd, s) ? EGEMM_ERR_CUDA : EGEMM_OK;
  int r;
  if ((r = check_operand(A, M, K, false, "A"))) return r;
  if ((r = check_operand(B, N, K, true, "B"))) return r;
  size_t need = gemm_operand_ws(M, N, K, A.hi != nullptr, B.hi != nullptr);
  if (need > 0 && (!workspace || workspace_bytes < need)) {
    set_last_error("workspace %zu < %zu", workspace_bytes, need);
    return EGEMM_ERR_WORKSPACE;
  }
  Carver cv{reinterpret_cast<char*>(workspace)};
  TcOperands ops = {};
  // B arriving as fp32 (either orientation): its split is part of this call -> "gemm_b32" rows
  TcConfig cfg = choose_config(EPI_STORE, M, N, K, terms, B.f32 && !B.hi);
  // fp32 row-major A (fa bit 0) or fp32 K x N row-major B (fa bit 1) can be round-split
  // inside the GEMM (converter warps, a-2 fused mode); B needs 16-B aligned rows (TMA)
  const bool fuse_a = (cfg.fa & 1) && !A.hi && !A.trans && fused_a_supported(cfg);
  const bool fuse_b = !fuse_a && (cfg.fa & 2) && !B.hi && B.f32 && !B.trans &&
                      fused_b_supported(cfg) && (B.ld % 4) == 0 &&
                      (reinterpret_cast<uintptr_t>(B.f32) % 16) == 0;
  if (fuse_a) {
    ops.a_f32 = A.f32;
    ops.lda_f32 = A.ld;
    cv.take<uint16_t>((size_t)(M * ldk_of(K)));  // keep B's workspace offset unchanged
    cv.take<uint16_t>((size_t)(M * ldk_of(K)));
  } else if ((r = stage_operand(A, M, K, cv, &ops.a_hi, &ops.a_lo, &ops.lda, s, cfg.fmt == 1 ? 2 : 0))) {
    return r;
  }
  // B logical K x N: as an operand it is N rows x K; f32 trans==0 means stored K x N.
  egemm_operand_t Bt = B;
  Bt.trans = !B.trans;
  if (fuse_b) {
    ops.b_f32 = B.f32;
    ops.ldb_f32 = B.ld;
    cv.take<uint16_t>((size_t)(N * ldk_of(K)));  // keep the workspace layout unchanged
    cv.take<uint16_t>((size_t)(N * ldk_of(K)));
  } else if ((r = stage_operand(Bt, N, K, cv, &ops.b_hi, &ops.b_lo, &ops.ldb, s, cfg.fmt == 1 ? 2 : 0,
                                /* B's split follows A's (independent) as its PDL dependent */
                                !fuse_a && !A.hi))) {
    return r;
  }
  TcEpilogue epi = {};
  epi.kind = EPI_STORE;
  epi.D = D;
  epi.ldd = ldd;
  epi.C = C;
  epi.ldc = ldc;
  if (const size_t pb = ksplit_ws_bytes(M, N, K, cfg)) {  // split-K parts buffer
    if (!workspace || workspace_bytes < cv.off + pb) {
      set_last_error("workspace %zu < %zu (split-K parts buffer; see egemm_gemm_workspace_size)",
                     workspace_bytes, cv.off + pb);
      return EGEMM_ERR_WORKSPACE;
    }
    epi.partial = cv.take<float>(pb / sizeof(float));
  } else if (const size_t tb = parts_ws_bytes(M, N, K, cfg)) {
    // tail split: optional -- without the room the last wave runs unsplit (same arithmetic
    // class; the split tiles follow R21's k-parts)
    if (workspace && workspace_bytes >= cv.off + tb + kPaceBytes) epi.partial = cv.take<float>(tb / sizeof(float));
  }
  if (workspace && workspace_bytes >= cv.off + kPaceBytes) epi.sync = cv.take<uint32_t>(64);
  r = launch_tc(M, N, K, ops, cfg, epi, s);
  return r == 0 ? EGEMM_OK : (r == 2 ? EGEMM_ERR_UNSUPPORTED : EGEMM_ERR_CUDA);
}

// ------------------------------------------------------------------ host-buffer GEMM
// D_host = A_host * B_host with the host<->device traffic pipelined against the compute:
// B is copied and split once, then row chunks of A flow H2D (copy stream) -> split ->
// tcgen05 GEMM (caller stream) -> D2H (second copy stream), double-buffered, so the two
// PCIe directions and the GPU work overlap.  Streams/events are created once per device.
static int64_t host_chunk_rows(int64_t M) {
  const int forced = knobs().host_chunk;  // experiments
  if (forced > 0) return forced > M ? M : forced;
  int64_t c = ((M / 8 + 255) / 256) * 256;
  if (c < 256) c = 256;
  if (c > 4096) c = 4096;
  return c > M ? M : c;
}

struct HostPipe {
  bool init = false;
  std::mutex mu;  // held by one call's whole enqueue sequence (the events are shared)
  cudaStream_t s_in = nullptr, s_out = nullptr;
  cudaEvent_t ev_start, ev_b, ev_in[2], ev_split[2], ev_comp[2], ev_out[2], ev_done;
};
static HostPipe g_pipe[64];
static std::mutex g_pipe_mu;

static HostPipe* host_pipe() {
  int dev = 0;
  if (cudaGetDevice(&dev) != cudaSuccess || dev < 0 || dev >= 64) return nullptr;
  std::lock_guard<std::mutex> lk(g_pipe_mu);
  HostPipe& p = g_pipe[dev];
  if (!p.init) {
    if (cudaStreamCreateWithFlags(&p.s_in, cudaStreamNonBlocking) != cudaSuccess ||
        cudaStreamCreateWithFlags(&p.s_out, cudaStreamNonBlocking) != cudaSuccess)
      return nullptr;
    // ev_done starts "complete" (recorded on an idle stream) so the first call's wait is free
    if (cudaEventCreateWithFlags(&p.ev_done, cudaEventDisableTiming) != cudaSuccess ||
        cudaEventRecord(p.ev_done, p.s_in) != cudaSuccess)
      return nullptr;
    cudaEvent_t* evs[] = {&p.ev_start, &p.ev_b, &p.ev_in[0], &p.ev_in[1], &p.ev_split[0],
                          &p.ev_split[1], &p.ev_comp[0], &p.ev_comp[1], &p.ev_out[0], &p.ev_out[1]};
    for (cudaEvent_t* e : evs)
      if (cudaEventCreateWithFlags(e, cudaEventDisableTiming) != cudaSuccess) return nullptr;
    p.init = true;
  }
  return &p;
}

size_t egemm_gemm_host_workspace_size(int64_t M, int64_t N, int64_t K) {
  if (M <= 0 || N <= 0 || K <= 0) return 0;
  const int64_t ldk = ldk_of(K), mc = host_chunk_rows(M);
  Carver cv{nullptr};
  cv.take<float>((size_t)(K * N));
  cv.take<uint16_t>((size_t)(N * ldk));
  cv.take<uint16_t>((size_t)(N * ldk));
  for (int b = 0; b < 2; b++) {
    cv.take<float>((size_t)(mc * K));
    cv.take<uint16_t>((size_t)(mc * ldk));
    cv.take<uint16_t>((size_t)(mc * ldk));
    cv.take<float>((size_t)(mc * N));
  }
  return cv.off;
}

int egemm_gemm_host(int64_t M, int64_t N, int64_t K, const float* A_host, int64_t lda,
                    const float* B_host, int64_t ldb, float* D_host, int64_t ldd, int terms,
                    void* workspace, size_t workspace_bytes, void* stream) {
  NvtxRange nvtx_range("egemm_gemm_host");
  cudaStream_t s = (cudaStream_t)stream;
  if (M < 0 || N < 0 || K < 0 || lda < K || ldb < N || ldd < N) {
    set_last_error("negative size or ld too small");
    return EGEMM_ERR_INVALID_ARG;
  }
  if (terms == 0) terms = 3;
  if (terms != 3 && terms != 4) {
    set_last_error("terms must be 0, 3 or 4");
    return EGEMM_ERR_INVALID_ARG;
  }
  if (M == 0 || N == 0) return EGEMM_OK;
  if (!A_host || !B_host || !D_host) {
    set_last_error("NULL host pointer");
    return EGEMM_ERR_INVALID_ARG;
  }
  if (K == 0) {
    set_last_error("K == 0: use egemm_gemm (nothing to stream)");
    return EGEMM_ERR_UNSUPPORTED;
  }
  if (!device_ok()) {
    set_last_error("no sm_100 device");
    return EGEMM_ERR_CUDA;
  }
  const size_t need = egemm_gemm_host_workspace_size(M, N, K);
  if (!workspace || workspace_bytes < need) {
    set_last_error("workspace %zu < %zu", workspace_bytes, need);
    return EGEMM_ERR_WORKSPACE;
  }
  HostPipe* hp = host_pipe();
  if (!hp) {
    set_last_error("stream/event creation failed");
    return EGEMM_ERR_CUDA;
  }
  // one call at a time per device: the pipeline's events are shared, and the copy streams
  // of this call must not start before the previous call (maybe from another thread, on
  // another stream) has finished with its buffers and events
  std::lock_guard<std::mutex> call_lock(hp->mu);
  const int64_t ldk = ldk_of(K), mc = host_chunk_rows(M);
  Carver cv{reinterpret_cast<char*>(workspace)};
  float* Bd = cv.take<float>((size_t)(K * N));
  uint16_t* bhi = cv.take<uint16_t>((size_t)(N * ldk));
  uint16_t* blo = cv.take<uint16_t>((size_t)(N * ldk));
  float* Ad[2];
  uint16_t *ahi[2], *alo[2];
  float* Dd[2];
  for (int b = 0; b < 2; b++) {
    Ad[b] = cv.take<float>((size_t)(mc * K));
    ahi[b] = cv.take<uint16_t>((size_t)(mc * ldk));
    alo[b] = cv.take<uint16_t>((size_t)(mc * ldk));
    Dd[b] = cv.take<float>((size_t)(mc * N));
  }
  TcConfig cfg = choose_config(EPI_STORE, mc, N, K, terms);
  cfg.ksplit = 0;  // (no parts buffer in the host pipeline's workspace)
  cfg.tsplit = 0;
  bool ok = true;
  auto chk = [&](cudaError_t e) { ok = ok && (e == cudaSuccess); };
  chk(cudaStreamWaitEvent(s, hp->ev_done, 0));  // the previous call's pipeline has drained
  chk(cudaEventRecord(hp->ev_start, s));
  chk(cudaStreamWaitEvent(hp->s_in, hp->ev_start, 0));
  chk(cudaStreamWaitEvent(hp->s_out, hp->ev_start, 0));
  chk(cudaMemcpy2DAsync(Bd, N * sizeof(float), B_host, ldb * sizeof(float), N * sizeof(float), K,
                        cudaMemcpyHostToDevice, hp->s_in));
  chk(cudaEventRecord(hp->ev_b, hp->s_in));
  chk(cudaStreamWaitEvent(s, hp->ev_b, 0));
  if (!ok || launch_split(Bd, K, N, N, bhi, blo, ldk, 1, nullptr, s)) {
    set_last_error("B staging failed");
    return EGEMM_ERR_CUDA;
  }
  const int64_t nchunks = (M + mc - 1) / mc;
  for (int64_t c = 0; c < nchunks && ok; c++) {
    const int b = (int)(c & 1);
    const int64_t r0 = c * mc, rows = (M - r0 < mc) ? M - r0 : mc;
    if (c >= 2) chk(cudaStreamWaitEvent(hp->s_in, hp->ev_split[b], 0));  // Ad[b] free
    chk(cudaMemcpy2DAsync(Ad[b], K * sizeof(float), A_host + r0 * lda, lda * sizeof(float),
                          K * sizeof(float), rows, cudaMemcpyHostToDevice, hp->s_in));
    chk(cudaEventRecord(hp->ev_in[b], hp->s_in));
    chk(cudaStreamWaitEvent(s, hp->ev_in[b], 0));
    const bool fuse_a = cfg.fa && fused_a_supported(cfg);
    if (!fuse_a) {
      if (launch_split(Ad[b], rows, K, K, ahi[b], alo[b], ldk, 0, nullptr, s)) ok = false;
      chk(cudaEventRecord(hp->ev_split[b], s));
    }
    if (c >= 2) chk(cudaStreamWaitEvent(s, hp->ev_out[b], 0));  // Dd[b] drained
    TcOperands ops = {ahi[b], alo[b], ldk, bhi, blo, ldk};
    if (fuse_a) {  // the GEMM's converter warps split A straight from Ad[b]
      ops.a_f32 = Ad[b];
      ops.lda_f32 = K;
    }
    TcEpilogue epi = {};
    epi.kind = EPI_STORE;
    epi.D = Dd[b];
    epi.ldd = N;
    if (ok && launch_tc(rows, N, K, ops, cfg, epi, s)) ok = false;
    if (fuse_a) chk(cudaEventRecord(hp->ev_split[b], s));  // Ad[b] consumed by the GEMM
    chk(cudaEventRecord(hp->ev_comp[b], s));
    chk(cudaStreamWaitEvent(hp->s_out, hp->ev_comp[b], 0));
    chk(cudaMemcpy2DAsync(D_host + r0 * ldd, ldd * sizeof(float), Dd[b], N * sizeof(float),
                          N * sizeof(float), rows, cudaMemcpyDeviceToHost, hp->s_out));
    chk(cudaEventRecord(hp->ev_out[b], hp->s_out));
  }
  // the caller's stream completes only after the last D2H
  chk(cudaStreamWaitEvent(s, hp->ev_out[(nchunks - 1) & 1], 0));
  if (nchunks >= 2) chk(cudaStreamWaitEvent(s, hp->ev_out[(nchunks - 2) & 1], 0));
  chk(cudaEventRecord(hp->ev_done, s));
  if (!ok) {
    set_last_error("host pipeline: %s", cudaGetErrorString(cudaGetLastError()));
    return EGEMM_ERR_CUDA;
  }
  return EGEMM_OK;
}

// N-slices per query block (wave balance over the persistent clusters); slices of the same
// rows share their k-th-key bound (row_bound), so later slices skip most of the warm-up.
constexpr int kKnnMaxSlices = 16;
static int knn_slices(int64_t nq, int64_t nx, int cg, int bn) {
  const int64_t m_tiles = (nq + 128 * cg - 1) / (128 * cg);
  const int64_t n_tiles = (nx + bn - 1) / bn;
  const int64_t clusters = num_sms() / cg > 0 ? num_sms() / cg : 1;
  int best = 1;
  double best_eff = 0.0;
  for (int s = 1; s <= kKnnMaxSlices && s <= n_tiles; s++) {
    int64_t units = m_tiles * s;
    int64_t waves = (units + clusters - 1) / clusters;
    double eff = (double)units / (double)(waves * clusters);
    if (eff >= 0.97) return s;
    if (eff > best_eff + 1e-9) { best_eff = eff; best = s; }
  }
  return best;
}

size_t egemm_knn_workspace_size(int64_t nx, int64_t nq, int64_t d, int k, int x_presplit) {
  if (nx <= 0 || nq <= 0 || d <= 0 || k <= 0) return 0;
  Carver cv{nullptr};
  const int64_t ldk = ldk_of(d);
  if (!x_presplit) { cv.take<uint16_t>((size_t)(nx * ldk)); cv.take<uint16_t>((size_t)(nx * ldk)); }
  cv.take<uint16_t>((size_t)(nq * ldk));
  cv.take<uint16_t>((size_t)(nq * ldk));
  cv.take<float>((size_t)nx);
  cv.take<float>((size_t)nq);
  cv.take<float>((size_t)(kKnnMaxSlices * nq * k));
  cv.take<int32_t>((size_t)(kKnnMaxSlices * nq * k));
  cv.take<float>((size_t)nq);
  return cv.off;
}

int egemm_knn_index(const float* X, int64_t nx, int64_t d, int64_t ldx, uint16_t* hi, uint16_t* lo,
                    int64_t ld_split, float* norms, void* stream) {
  NvtxRange nvtx_range("egemm_knn_index");
  cudaStream_t s = (cudaStream_t)stream;
  if (nx < 0 || d <= 0 || ldx < d || ld_split < d || (ld_split % 8) != 0) {
    set_last_error("need nx >= 0, d > 0, ldx >= d, ld_split >= d and a multiple of 8");
    return EGEMM_ERR_INVALID_ARG;
  }
  if (nx == 0) return EGEMM_OK;
  if (!X || !hi || !lo || !norms) {
    set_last_error("NULL pointer");
    return EGEMM_ERR_INVALID_ARG;
  }
  if (!device_ok()) {
    set_last_error("no sm_100 device");
    return EGEMM_ERR_CUDA;
  }
  if (launch_split(X, nx, d, ldx, hi, lo, ld_split, 0, nullptr, s) ||
      launch_rownorm(X, nx, d, ldx, norms, s))
    return EGEMM_ERR_CUDA;
  return EGEMM_OK;
}

int egemm_knn(egemm_operand_t X, const float* x_norms, int64_t nx, egemm_operand_t Q, int64_t nq,
              int64_t d, int k, int32_t* out_idx, float* out_dist, void* workspace,
              size_t workspace_bytes, void* stream) {
  NvtxRange nvtx_range("egemm_knn");
  cudaStream_t s = (cudaStream_t)stream;
  if (nx < 0 || nq < 0 || d <= 0 || k < 1 || k > 64 || k > nx) {
    set_last_error("need nx, nq >= 0, d > 0, 1 <= k <= min(64, nx)");
    return EGEMM_ERR_INVALID_ARG;
  }
  if (nq == 0) return EGEMM_OK;
  if ((!X.f32 && !x_norms) || !Q.f32 || X.trans || Q.trans || (X.f32 && X.ld < d) || Q.ld < d ||
      !out_idx || !out_dist) {
    set_last_error("X needs fp32 rows or (hi/lo + x_norms); Q fp32 rows (trans 0, ld >= d)");
    return EGEMM_ERR_INVALID_ARG;
  }
  if (!X.f32 && !(X.hi && X.lo)) {
    set_last_error("X: no data");
    return EGEMM_ERR_INVALID_ARG;
  }
  if (d > 1024) {
    set_last_error("d > 1024 not supported by the fused epilogue");
    return EGEMM_ERR_UNSUPPORTED;
  }
  if (!device_ok()) {
    set_last_error("no sm_100 device");
    return EGEMM_ERR_CUDA;
  }
  int r;
  if ((r = check_operand(X, nx, d, false, "X"))) return r;
  size_t need = egemm_knn_workspace_size(nx, nq, d, k, X.hi != nullptr);
  if (!workspace || workspace_bytes < need) {
    set_last_error("workspace %zu < %zu", workspace_bytes, need);
    return EGEMM_ERR_WORKSPACE;
  }
  TcConfig cfg = choose_config(EPI_KNN, nq, nx, d, 3);
  Carver cv{reinterpret_cast<char*>(workspace)};
  TcOperands ops = {};
  if ((r = stage_operand(X, nx, d, cv, &ops.b_hi, &ops.b_lo, &ops.ldb, s))) return r;
  egemm_operand_t Qs = Q;
  Qs.hi = Qs.lo = nullptr;
  if ((r = stage_operand(Qs, nq, d, cv, &ops.a_hi, &ops.a_lo, &ops.lda, s))) return r;
  float* xnorm = cv.take<float>((size_t)nx);
  float* qnorm = cv.take<float>((size_t)nq);
  float* pkey = cv.take<float>((size_t)(kKnnMaxSlices * nq * k));
  int32_t* pidx = cv.take<int32_t>((size_t)(kKnnMaxSlices * nq * k));
  float* rbound = cv.take<float>((size_t)nq);
  if (cudaMemsetAsync(rbound, 0xFF, sizeof(float) * (size_t)nq, s) != cudaSuccess) {
    set_last_error("memset of the row bounds failed");
    return EGEMM_ERR_CUDA;
  }
  if (x_norms) xnorm = const_cast<float*>(x_norms);
  else if (launch_rownorm(X.f32, nx, d, X.ld, xnorm, s)) return EGEMM_ERR_CUDA;
  if (launch_rownorm(Q.f32, nq, d, Q.ld, qnorm, s)) return EGEMM_ERR_CUDA;
  TcEpilogue epi = {};
  epi.kind = EPI_KNN;
  epi.bnorm = xnorm;
  epi.knn_k = k;
  {
    const int64_t n_tiles = (nx + cfg.bn - 1) / cfg.bn;
    int ns = cfg.nslices > 0 ? cfg.nslices : knn_slices(nq, nx, cfg.cg, cfg.bn);
    if (ns > kKnnMaxSlices) ns = kKnnMaxSlices;
    if (ns > n_tiles) ns = (int)n_tiles;
    epi.n_slices = ns < 1 ? 1 : ns;
  }
  epi.row_bound = rbound;
  epi.part_key = pkey;
  epi.part_idx = pidx;
  r = launch_tc(nq, nx, d, ops, cfg, epi, s);
  if (r) return r == 2 ? EGEMM_ERR_UNSUPPORTED : EGEMM_ERR_CUDA;
  if (launch_knn_merge(pkey, pidx, epi.n_slices, nq, k, k, qnorm, out_idx, out_dist, s))
    return EGEMM_ERR_CUDA;
  return EGEMM_OK;
}

int egemm_knn_merge(const float* keys, const int32_t* idx, int n_lists, int64_t nq, int k_in, int k,
                    const float* qnorm, int32_t* out_idx, float* out_key, void* stream) {
  NvtxRange nvtx_range("egemm_knn_merge");
  if (nq < 0 || n_lists < 1 || n_lists > 64 || k_in < 1 || k_in > 1024 || k < 1 || k > 64 ||
      (int64_t)k > (int64_t)k_in * n_lists) {
    set_last_error("need nq >= 0, 1 <= n_lists <= 64, 1 <= k_in <= 1024, 1 <= k <= min(64, k_in * n_lists)");
    return EGEMM_ERR_INVALID_ARG;
  }
  if (nq == 0) return EGEMM_OK;
  if (!keys || !idx || !out_idx || !out_key) {
    set_last_error("NULL pointer");
    return EGEMM_ERR_INVALID_ARG;
  }
  if (!device_ok()) {
    set_last_error("no sm_100 device");
    return EGEMM_ERR_CUDA;
  }
  return launch_knn_merge(keys, idx, n_lists, nq, k_in, k, qnorm, out_idx, out_key,
                          (cudaStream_t)stream)
             ? EGEMM_ERR_CUDA
             : EGEMM_OK;
}

size_t egemm_kmeans_workspace_size(int64_t n, int64_t d, int64_t kc, int x_presplit) {
  if (n <= 0 || d <= 0 || kc <= 0) return 0;
  Carver cv{nullptr};
  const int64_t ldk = ldk_of(d);
  if (!x_presplit) { cv.take<uint16_t>((size_t)(n * ldk)); cv.take<uint16_t>((size_t)(n * ldk)); }
  cv.take<uint16_t>((size_t)(kc * ldk));
  cv.take<uint16_t>((size_t)(kc * ldk));
  cv.take<float>((size_t)kc);
  cv.take<float>((size_t)n);
  cv.take<char>(kmeans_accumulate_ws(n, d, kc));
  return cv.off;
}

int egemm_kmeans_step(egemm_operand_t X, int64_t n, int64_t d, const float* centroids, int64_t kc,
                      int32_t* assign, double* sums, int64_t* counts, double* inertia,
                      void* workspace, size_t workspace_bytes, void* stream) {
  NvtxRange nvtx_range("egemm_kmeans_step");
  cudaStream_t s = (cudaStream_t)stream;
  if (n < 0 || d <= 0 || kc <= 0 || !centroids || !assign || !sums || !counts) {
    set_last_error("need n >= 0, d > 0, kc > 0 and non-NULL centroids/assign/sums/counts");
    return EGEMM_ERR_INVALID_ARG;
  }
  if (!X.f32 || X.trans || X.ld < d) {
    set_last_error("X needs fp32 rows (trans 0, ld >= d)");
    return EGEMM_ERR_INVALID_ARG;
  }
  if (d > 1024 || kc > 12288) {
    set_last_error("d > 1024 or kc > 12288 not supported by the fused epilogue / sums");
    return EGEMM_ERR_UNSUPPORTED;
  }
  if (!device_ok()) {
    set_last_error("no sm_100 device");
    return EGEMM_ERR_CUDA;
  }
  int r;
  if ((r = check_operand(X, n, d, false, "X"))) return r;
  size_t need = egemm_kmeans_workspace_size(n, d, kc, X.hi != nullptr);
  if (n > 0 && (!workspace || workspace_bytes < need)) {
    set_last_error("workspace %zu < %zu", workspace_bytes, need);
    return EGEMM_ERR_WORKSPACE;
  }
  if (n == 0)
    return launch_kmeans_accumulate(nullptr, 0, d, d, nullptr, nullptr, kc, sums, counts, inertia,
                                    nullptr, s)
               ? EGEMM_ERR_CUDA
               : EGEMM_OK;
  TcConfig cfg = choose_config(EPI_KMEANS, n, kc, d, 3);
  Carver cv{reinterpret_cast<char*>(workspace)};
  TcOperands ops = {};
  if ((r = stage_operand(X, n, d, cv, &ops.a_hi, &ops.a_lo, &ops.lda, s))) return r;
  egemm_operand_t Cop = {centroids, nullptr, nullptr, d, 0, 0};
  if ((r = stage_operand(Cop, kc, d, cv, &ops.b_hi, &ops.b_lo, &ops.ldb, s))) return r;
  float* cnorm = cv.take<float>((size_t)kc);
  float* best = cv.take<float>((size_t)n);
  void* accws = cv.take<char>(kmeans_accumulate_ws(n, d, kc));
  if (launch_rownorm(centroids, kc, d, d, cnorm, s)) return EGEMM_ERR_CUDA;
  TcEpilogue epi = {};
  epi.kind = EPI_KMEANS;
  epi.bnorm = cnorm;
  epi.assign = assign;
  epi.best_key = best;
  r = launch_tc(n, kc, d, ops, cfg, epi, s);
  if (r) return r == 2 ? EGEMM_ERR_UNSUPPORTED : EGEMM_ERR_CUDA;
  r = launch_kmeans_accumulate(X.f32, n, d, X.ld, assign, best, kc, sums, counts, inertia, accws, s);
  return r == 0 ? EGEMM_OK : (r == 2 ? EGEMM_ERR_UNSUPPORTED : EGEMM_ERR_CUDA);
}

int egemm_kmeans_finalize(const double* sums, const int64_t* counts, int64_t kc, int64_t d,
                          float* centroids, void* stream) {
  NvtxRange nvtx_range("egemm_kmeans_finalize");
  if (kc < 0 || d < 0 || (kc * d > 0 && (!sums || !counts || !centroids))) {
    set_last_error("bad kmeans_finalize arguments");
    return EGEMM_ERR_INVALID_ARG;
  }
  if (!device_ok()) {
    set_last_error("no sm_100 device");
    return EGEMM_ERR_CUDA;
  }
  return launch_kmeans_finalize(sums, counts, kc, d, centroids, (cudaStream_t)stream)
             ? EGEMM_ERR_CUDA
             : EGEMM_OK;
}

int egemm_kmeans_allreduce_finalize(const double* const* peer_sums,
                                    const int64_t* const* peer_counts, int nranks, int64_t kc,
                                    int64_t d, double* sums_out, int64_t* counts_out,
                                    float* centroids, void* stream) {
  NvtxRange nvtx_range("egemm_kmeans_allreduce_finalize");
  if (nranks < 1 || nranks > kMaxPeers || kc < 0 || d < 0 || !peer_sums || !peer_counts ||
      (kc * d > 0 && !centroids)) {
    set_last_error("need 1 <= nranks <= %d, host arrays of peer pointers, centroids", kMaxPeers);
    return EGEMM_ERR_INVALID_ARG;
  }
  for (int r = 0; r < nranks; r++)
    if (!peer_sums[r] || !peer_counts[r]) {
      set_last_error("peer %d: NULL buffer", r);
      return EGEMM_ERR_INVALID_ARG;
    }
  if (!device_ok()) {
    set_last_error("no sm_100 device");
    return EGEMM_ERR_CUDA;
  }
  return launch_kmeans_peer_reduce_finalize(peer_sums, peer_counts, nranks, kc, d, sums_out,
                                            counts_out, centroids, (cudaStream_t)stream)
             ? EGEMM_ERR_CUDA
             : EGEMM_OK;
}

}  // extern "C"
