// kmeans.cu -- kMeans centroid partial sums / counts / inertia after the tensor-core
// assignment step (the GEMM-based kMeans of [2]), and
// the centroid update.
//
// Sums are fp64 and deterministic, in the fixed two-level order of reading R20:
//   the members of group j (points with a_i == j) in ascending i are cut into chunks of
//   kKmChunk; each chunk is summed sequentially from 0.0; the chunk sums are then added
//   sequentially from 0.0.  tests/kernel_model.py (group_sums_chunked) models this order
//   for the bitwise regression test; the oracle sums each group plainly in ascending i
//   (SURVEY c-6) and the GPU sums are checked against it within the fp64 sum bound.
// Instead of 4M x 64 fp64 atomics (measured 1.9 ms) a stable counting sort groups the
// point indices by centroid, then one CTA per chunk (one thread per dimension) adds rows
// gathered 32 at a time, and one CTA per centroid adds its chunk sums:
//   A  km_hist       per-block histogram H[j][b] (smem atomics)
//   B1 km_scan_blk   per-centroid exclusive scan over blocks, cnt[j]
//   B2 km_scan_c     offsets[j], counts[j], chunk_base[j], chunk -> centroid map
//   C  km_scatter    stable scatter: the block's 4096 points in W warp sub-ranges, per-warp
//                    histograms -> per-warp offsets, then in-warp ranks from per-bit ballots
//   D  km_chunk      chunk partial sums (+ per-chunk inertia terms); the CTA that finishes
//                    the last chunk of centroid j (atomic ticket) adds j's chunk partials in
//                    chunk order: sums[j] (+ inertia_j) -- the old separate combine pass
//   F  km_inertia    inertia = fixed-order tree sum of inertia_j
#include <cuda_runtime.h>
#include <cstdint>
#include "egemm_internal.h"

namespace egemm {

constexpr int kKmBlockPts = 4096;  // points per histogram / scatter block
constexpr int kKmChunk = 256;      // rows per chunk partial sum (reading R20)

__global__ void km_hist_kernel(const int32_t* __restrict__ assign, int64_t n, int64_t kc,
                               int32_t* __restrict__ H, int nb) {
  extern __shared__ int32_t h[];
  for (int64_t j = threadIdx.x; j < kc; j += blockDim.x) h[j] = 0;
  __syncthreads();
  const int64_t i0 = (int64_t)blockIdx.x * kKmBlockPts;
  const int64_t i1 = min(n, i0 + kKmBlockPts);
  for (int64_t i = i0 + threadIdx.x; i < i1; i += blockDim.x) atomicAdd(&h[assign[i]], 1);
  __syncthreads();
  for (int64_t j = threadIdx.x; j < kc; j += blockDim.x) H[j * nb + blockIdx.x] = h[j];
}

// block-wide exclusive scan helper (blockDim multiple of 32, <= 1024); returns the
// exclusive prefix of v and writes the block total to *total.
template <class T>
__device__ __forceinline__ T block_excl_scan(T v, T* warp_tot, T* total) {
  T x = v;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    T y = __shfl_up_sync(0xffffffffu, x, o);
    if ((threadIdx.x & 31) >= (unsigned)o) x += y;
  }
  if ((threadIdx.x & 31) == 31) warp_tot[threadIdx.x >> 5] = x;
  __syncthreads();
  T wpre = 0, tot = 0;
  for (int w = 0; w < (int)(blockDim.x >> 5); w++) {
    if (w < (int)(threadIdx.x >> 5)) wpre += warp_tot[w];
    tot += warp_tot[w];
  }
  __syncthreads();
  *total = tot;
  return wpre + x - v;
}

__global__ void km_scan_blk_kernel(int32_t* __restrict__ H, int nb, int32_t* __restrict__ cnt) {
  __shared__ int32_t warp_tot[32];
  int32_t* row = H + (int64_t)blockIdx.x * nb;
  int32_t carry = 0;
  for (int base = 0; base < nb; base += blockDim.x) {
    const int b = base + threadIdx.x;
    const int32_t v = b < nb ? row[b] : 0;
    int32_t tot;
    const int32_t ex = block_excl_scan<int32_t>(v, warp_tot, &tot);
    if (b < nb) row[b] = carry + ex;
    carry += tot;
  }
  if (threadIdx.x == 0) cnt[blockIdx.x] = carry;
}

__global__ void km_scan_c_kernel(const int32_t* __restrict__ cnt, int64_t kc,
                                 int64_t* __restrict__ offsets, int64_t* __restrict__ counts,
                                 int32_t* __restrict__ chunk_base, int32_t* __restrict__ chunk_j,
                                 int32_t* __restrict__ n_chunks, int32_t* __restrict__ done,
                                 double* __restrict__ sums, int64_t d, double* __restrict__ in_j) {
  __shared__ int64_t wt64[32];
  __shared__ int32_t wt32[32];
  int64_t carry = 0;
  int32_t ccarry = 0;
  for (int64_t base = 0; base < kc; base += blockDim.x) {
    const int64_t j = base + threadIdx.x;
    const int32_t c = j < kc ? cnt[j] : 0;
    const int32_t nch = (c + kKmChunk - 1) / kKmChunk;
    int64_t tot;
    int32_t ctot;
    const int64_t ex = block_excl_scan<int64_t>((int64_t)c, wt64, &tot);
    const int32_t cex = block_excl_scan<int32_t>(nch, wt32, &ctot);
    if (j < kc) {
      offsets[j] = carry + ex;
      counts[j] = c;
      chunk_base[j] = ccarry + cex;
      done[j] = 0;  // km_chunk's per-centroid tickets
      if (c == 0) {  // no chunk will write an empty cluster's sums
        for (int64_t t = 0; t < d; t++) sums[j * d + t] = 0.0;
        in_j[j] = 0.0;
      }
      for (int32_t q = 0; q < nch; q++) chunk_j[ccarry + cex + q] = (int32_t)j;
    }
    carry += tot;
    ccarry += ctot;
  }
  if (threadIdx.x == 0) *n_chunks = ccarry;
}

// Stable scatter of one block of kKmBlockPts points: W warps take consecutive sub-ranges;
// pass 1 counts each warp's members per centroid (peer lanes by ballots: the leader of each group
// adds its popcount, so no atomics), the counts become per-warp start offsets (block base
// H[a][b] + earlier warps), pass 2 writes order[] with the in-warp ranks.  Same positions as
// a sequential walk over the block: the order stays stable (ascending i per centroid).
// Lanes of the warp holding the same centroid as this lane (valid lanes only): one ballot
// per bit of the centroid index instead of __match_any_sync, whose result latency bounded the
// scatter (ncu: the stalls sat on the instructions consuming MATCH).
__device__ __forceinline__ uint32_t same_key_lanes(int a, bool valid, int nbits) {
  uint32_t m = __ballot_sync(0xffffffffu, valid);
  for (int b = 0; b < nbits; b++) {
    const bool bit = (a >> b) & 1;
    const uint32_t bb = __ballot_sync(0xffffffffu, bit);
    m &= bit ? bb : ~bb;
  }
  return m;
}

template <int W>
__global__ void __launch_bounds__(32 * W) km_scatter_kernel(
    const int32_t* __restrict__ assign, int64_t n, int64_t kc, const int32_t* __restrict__ H,
    int nb, const int64_t* __restrict__ offsets, int32_t* __restrict__ order) {
  extern __shared__ int32_t hw[];  // [W][kc]
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  for (int64_t j = threadIdx.x; j < (int64_t)W * kc; j += blockDim.x) hw[j] = 0;
  __syncthreads();
  const int64_t i0 = (int64_t)blockIdx.x * kKmBlockPts;
  const int64_t i1 = min(n, i0 + kKmBlockPts);
  constexpr int SUB = kKmBlockPts / W;
  constexpr int B = 16;  // assignments held in registers per lane (the loads of a batch overlap)
  const int64_t s0 = i0 + (int64_t)w * SUB, s1 = min(i1, s0 + SUB);
  int32_t* mine = hw + (int64_t)w * kc;
  const int nbits = kc > 1 ? 32 - __clz((int)(kc - 1)) : 0;
  // KEEP (one batch per warp, W = 8): the batch's keys and peer masks stay in registers for
  // pass 2 instead of being loaded and recomputed (the ballots are most of the kernel's work)
  constexpr bool KEEP = (SUB == 32 * B);
  int kav[KEEP ? B : 1];
  uint32_t kpeers[KEEP ? B : 1];
  for (int64_t cb = s0; cb < s1; cb += 32 * B) {
    int av[B];
#pragma unroll
    for (int t = 0; t < B; t++) {
      const int64_t i = cb + 32 * t + lane;
      av[t] = i < s1 ? assign[i] : 0;
    }
#pragma unroll
    for (int t = 0; t < B; t++) {
      const int64_t i = cb + 32 * t + lane;
      const uint32_t peers = same_key_lanes(av[t], i < s1, nbits);
      if (i < s1 && lane == __ffs(peers) - 1) mine[av[t]] += __popc(peers);
      if constexpr (KEEP) { kav[t] = av[t]; kpeers[t] = peers; }
      __syncwarp();  // the next batch's leader of this centroid may be another lane
    }
  }
  __syncthreads();
  // exclusive prefix over warps, starting at the centroid's global offset plus the counts of
  // the earlier blocks: hw then holds each warp's first output position per centroid
  for (int64_t j = threadIdx.x; j < kc; j += blockDim.x) {
    int32_t run = (int32_t)offsets[j] + H[j * nb + blockIdx.x];
#pragma unroll
    for (int v = 0; v < W; v++) {
      const int32_t t = hw[(int64_t)v * kc + j];
      hw[(int64_t)v * kc + j] = run;
      run += t;
    }
  }
  __syncthreads();
  for (int64_t cb = s0; cb < s1; cb += 32 * B) {
    int av[B];
    if constexpr (!KEEP) {
#pragma unroll
      for (int t = 0; t < B; t++) {
        const int64_t i = cb + 32 * t + lane;
        av[t] = i < s1 ? assign[i] : 0;
      }
    }
#pragma unroll
    for (int t = 0; t < B; t++) {
      const int64_t i = cb + 32 * t + lane;
      const bool valid = i < s1;
      const int a = KEEP ? kav[t] : av[t];
      const uint32_t peers = KEEP ? kpeers[t] : same_key_lanes(a, valid, nbits);
      const int rank = __popc(peers & ((1u << lane) - 1u));
      if (valid) order[mine[a] + rank] = (int32_t)i;
      __syncwarp();
      if (valid && lane == __ffs(peers) - 1) mine[a] += __popc(peers);
      __syncwarp();
    }
  }
}

// one CTA per chunk g, one thread per dimension (blockDim >= d): sequential fp64 chunk
// sum over <= kKmChunk rows, gathered 32 rows at a time.
__global__ void km_chunk_kernel(const float* __restrict__ X, int64_t d, int64_t ldx,
                                const int32_t* __restrict__ order,
                                const int64_t* __restrict__ offsets,
                                const int64_t* __restrict__ counts,
                                const int32_t* __restrict__ chunk_base,
                                const int32_t* __restrict__ chunk_j,
                                const int32_t* __restrict__ n_chunks,
                                const float* __restrict__ best_key, double* __restrict__ part,
                                double* __restrict__ part_in, int32_t* __restrict__ done,
                                double* __restrict__ sums, double* __restrict__ in_j) {
  __shared__ int32_t sidx[kKmChunk];
  __shared__ double red[32];
  __shared__ int last;
  const int g = blockIdx.x;
  if (g >= *n_chunks) return;
  const int j = chunk_j[g];
  const int64_t c0 = (int64_t)(g - chunk_base[j]) * kKmChunk;
  const int nrow = (int)min((int64_t)kKmChunk, counts[j] - c0);
  const int32_t* ord = order + offsets[j] + c0;
  for (int r = threadIdx.x; r < nrow; r += blockDim.x) sidx[r] = ord[r];
  __syncthreads();
  const int64_t t = threadIdx.x;
  const bool active = t < d;
  double s = 0.0, q = 0.0;
  for (int r0 = 0; r0 < nrow; r0 += 32) {
    float xv[32];
#pragma unroll
    for (int r = 0; r < 32; r++)
      xv[r] = (active && r0 + r < nrow) ? __ldg(X + (int64_t)sidx[r0 + r] * ldx + t) : 0.f;
#pragma unroll
    for (int r = 0; r < 32; r++) {
      if (r0 + r < nrow) {
        s = __dadd_rn(s, (double)xv[r]);
        q = __fma_rn((double)xv[r], (double)xv[r], q);
      }
    }
  }
  if (active) part[(int64_t)g * d + t] = s;
  if (part_in) {
    // inertia terms of this chunk: sum over dims of x^2 plus the rows' best keys, in a
    // fixed order (warp shuffle tree, then warps in order) -> deterministic
    double v = active ? q : 0.0;
    for (int r = threadIdx.x; r < nrow; r += blockDim.x) v += (double)best_key[sidx[r]];
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    if ((threadIdx.x & 31) == 0) red[threadIdx.x >> 5] = v;
    __syncthreads();
    if (threadIdx.x == 0) {
      double w = 0.0;
      for (int k = 0; k < (int)(blockDim.x >> 5); k++) w += red[k];
      part_in[g] = w;
    }
  }
  // The CTA that completes centroid j's last chunk adds j's chunk partials in chunk order
  // (R20's second level): which CTA does it does not change the order or the bits.
  const int nch = (int)((counts[j] + kKmChunk - 1) / kKmChunk);
  __threadfence();  // this thread's partials before the ticket
  __syncthreads();
  if (threadIdx.x == 0) {
    last = (atomicAdd(done + j, 1) == nch - 1);
    __threadfence();
  }
  __syncthreads();
  if (!last) return;
  const int64_t g0 = chunk_base[j];
  if (active) {
    double acc = 0.0;
    for (int c = 0; c < nch; c++) acc = __dadd_rn(acc, __ldcg(part + (g0 + c) * d + t));
    sums[j * d + t] = acc;
  }
  if (part_in && threadIdx.x == 0) {
    double w = 0.0;
    for (int c = 0; c < nch; c++) w += __ldcg(part_in + g0 + c);
    in_j[j] = w;
  }
}

// The same chunk sums with float4 rows: a sub-group of TPC = d / 4 lanes (1 .. 32, inside one
// warp) takes one chunk, each lane 4 dimensions, 8 chunks per CTA.  Per dimension the rows are
// still added one by one in the chunk's order from 0.0 (R20), so the partials are bitwise those
// of km_chunk_kernel; a lane now keeps 4 independent fp64 chains and issues one 16-B load per
// row instead of four 4-B loads (the scalar kernel was issue-bound: ~26 instructions per
// element, 68 % issue utilisation).
constexpr int kKmVecChunks = 8;
template <bool INERTIA>
__global__ void km_chunk_vec_kernel(const float* __restrict__ X, int64_t d, int64_t ldx,
                                    const int32_t* __restrict__ order,
                                    const int64_t* __restrict__ offsets,
                                    const int64_t* __restrict__ counts,
                                    const int32_t* __restrict__ chunk_base,
                                    const int32_t* __restrict__ chunk_j,
                                    const int32_t* __restrict__ n_chunks,
                                    const float* __restrict__ best_key, double* __restrict__ part,
                                    double* __restrict__ part_in, int32_t* __restrict__ done,
                                    double* __restrict__ sums, double* __restrict__ in_j, int tpc_log2) {
  __shared__ int32_t sidx[kKmVecChunks][kKmChunk];
  const int tpc = 1 << tpc_log2;
  const int sub = (int)threadIdx.x >> tpc_log2;
  const int lt = (int)threadIdx.x & (tpc - 1);
  const int g = (int)blockIdx.x * kKmVecChunks + sub;
  const bool valid = g < *n_chunks;
  int j = 0, nrow = 0;
  int64_t c0 = 0;
  if (valid) {
    j = chunk_j[g];
    c0 = (int64_t)(g - chunk_base[j]) * kKmChunk;
    nrow = (int)min((int64_t)kKmChunk, counts[j] - c0);
    const int32_t* ord = order + offsets[j] + c0;
    for (int r = lt; r < nrow; r += tpc) sidx[sub][r] = ord[r];
  }
  __syncthreads();
  const int32_t* si = sidx[sub];
  const float4* X4 = reinterpret_cast<const float4*>(X) + lt;
  const int64_t ld4 = ldx >> 2;
  double s[4] = {0.0, 0.0, 0.0, 0.0}, q[4] = {0.0, 0.0, 0.0, 0.0};
  int r = 0;
  for (; r + 8 <= nrow; r += 8) {
    float4 v[8];
#pragma unroll
    for (int i = 0; i < 8; i++) v[i] = __ldg(X4 + (int64_t)si[r + i] * ld4);
#pragma unroll
    for (int i = 0; i < 8; i++) {
      const double a[4] = {(double)v[i].x, (double)v[i].y, (double)v[i].z, (double)v[i].w};
#pragma unroll
      for (int k = 0; k < 4; k++) {
        s[k] = __dadd_rn(s[k], a[k]);
        if (INERTIA) q[k] = __fma_rn(a[k], a[k], q[k]);
      }
    }
  }
  for (; r < nrow; r++) {
    const float4 v = __ldg(X4 + (int64_t)si[r] * ld4);
    const double a[4] = {(double)v.x, (double)v.y, (double)v.z, (double)v.w};
#pragma unroll
    for (int k = 0; k < 4; k++) {
      s[k] = __dadd_rn(s[k], a[k]);
      if (INERTIA) q[k] = __fma_rn(a[k], a[k], q[k]);
    }
  }
  double* pg = part + (int64_t)g * d + 4 * lt;
  if (valid) {
    reinterpret_cast<double2*>(pg)[0] = make_double2(s[0], s[1]);
    reinterpret_cast<double2*>(pg)[1] = make_double2(s[2], s[3]);
  }
  // sub-group lanes [sub * tpc, sub * tpc + tpc) of this warp
  const int wl = (int)threadIdx.x & 31;
  const int lead = wl & ~(tpc - 1);
  const unsigned wmask = blockDim.x >= 32 ? 0xffffffffu : ((1u << blockDim.x) - 1u);
  if (INERTIA) {
    // fixed-order inertia terms: the lane's 4 dims, its strided share of the rows' best keys,
    // then an xor tree over the sub-group (deterministic; compared to the oracle within 1e-5)
    double w = (q[0] + q[1]) + (q[2] + q[3]);
    for (int rr = lt; rr < nrow; rr += tpc) w += (double)best_key[si[rr]];
    for (int o = tpc >> 1; o > 0; o >>= 1) w += __shfl_xor_sync(wmask, w, o);
    if (valid && lt == 0) part_in[g] = w;
  }
  // the lane that completes centroid j's last chunk adds j's chunk partials in chunk order
  // (R20's second level) -- as in km_chunk_kernel
  const int nch = valid ? (int)((counts[j] + kKmChunk - 1) / kKmChunk) : 0;
  __threadfence();
  int last = 0;
  if (valid && lt == 0) {
    last = (atomicAdd(done + j, 1) == nch - 1);
    __threadfence();
  }
  last = __shfl_sync(wmask, last, lead);
  if (!valid || !last) return;
  const int64_t g0 = chunk_base[j];
  double acc[4] = {0.0, 0.0, 0.0, 0.0};
  for (int c = 0; c < nch; c++) {
    const double2* pp = reinterpret_cast<const double2*>(part + (g0 + c) * d + 4 * lt);
    const double2 a0 = __ldcg(pp), a1 = __ldcg(pp + 1);
    acc[0] = __dadd_rn(acc[0], a0.x);
    acc[1] = __dadd_rn(acc[1], a0.y);
    acc[2] = __dadd_rn(acc[2], a1.x);
    acc[3] = __dadd_rn(acc[3], a1.y);
  }
  double2* sj = reinterpret_cast<double2*>(sums + (int64_t)j * d + 4 * lt);
  sj[0] = make_double2(acc[0], acc[1]);
  sj[1] = make_double2(acc[2], acc[3]);
  if (INERTIA && lt == 0) {
    double w = 0.0;
    for (int c = 0; c < nch; c++) w += __ldcg(part_in + g0 + c);
    in_j[j] = w;
  }
}

__global__ void km_inertia_kernel(const double* __restrict__ in_j, int64_t kc,
                                  double* __restrict__ inertia) {
  __shared__ double red[1024];
  double v = 0.0;
  for (int64_t j = threadIdx.x; j < kc; j += blockDim.x) v += in_j[j];
  red[threadIdx.x] = v;
  __syncthreads();
  for (int s = blockDim.x / 2; s > 0; s >>= 1) {
    if ((int)threadIdx.x < s) red[threadIdx.x] += red[threadIdx.x + s];
    __syncthreads();
  }
  if (threadIdx.x == 0) *inertia = red[0];
}

struct KmWs {
  int32_t *H, *cnt, *chunk_base, *chunk_j, *n_chunks, *order, *done;
  int64_t* offsets;
  double *part, *part_in, *in_j;
};

static size_t al256(size_t x) { return (x + 255) & ~size_t(255); }

static KmWs carve(void* base, int64_t n, int64_t d, int64_t kc, size_t* total) {
  const int64_t nb = (n + kKmBlockPts - 1) / kKmBlockPts;
  const int64_t gmax = n / kKmChunk + kc + 1;  // sum_j ceil(cnt_j / chunk) <= n/chunk + kc
  KmWs w = {};
  char* p = reinterpret_cast<char*>(base);
  size_t off = 0;
  auto take = [&](size_t bytes) -> char* {
    char* r = p ? p + off : nullptr;
    off += al256(bytes);
    return r;
  };
  w.H = reinterpret_cast<int32_t*>(take(sizeof(int32_t) * (size_t)(kc * (nb > 0 ? nb : 1))));
  w.cnt = reinterpret_cast<int32_t*>(take(sizeof(int32_t) * (size_t)kc));
  w.chunk_base = reinterpret_cast<int32_t*>(take(sizeof(int32_t) * (size_t)kc));
  w.chunk_j = reinterpret_cast<int32_t*>(take(sizeof(int32_t) * (size_t)gmax));
  w.n_chunks = reinterpret_cast<int32_t*>(take(sizeof(int32_t)));
  w.done = reinterpret_cast<int32_t*>(take(sizeof(int32_t) * (size_t)kc));
  w.order = reinterpret_cast<int32_t*>(take(sizeof(int32_t) * (size_t)(n > 0 ? n : 1)));
  w.offsets = reinterpret_cast<int64_t*>(take(sizeof(int64_t) * (size_t)kc));
  w.part = reinterpret_cast<double*>(take(sizeof(double) * (size_t)(gmax * d)));
  w.part_in = reinterpret_cast<double*>(take(sizeof(double) * (size_t)gmax));
  w.in_j = reinterpret_cast<double*>(take(sizeof(double) * (size_t)kc));
  *total = off;
  return w;
}

size_t kmeans_accumulate_ws(int64_t n, int64_t d, int64_t kc) {
  size_t total = 0;
  carve(nullptr, n, d, kc, &total);
  return total;
}

int launch_kmeans_accumulate(const float* X, int64_t n, int64_t d, int64_t ldx,
                             const int32_t* assign, const float* best_key, int64_t kc, double* sums,
                             int64_t* counts, double* inertia, void* ws, cudaStream_t stream) {
  if (n <= 0) {
    if (cudaMemsetAsync(sums, 0, sizeof(double) * (size_t)(kc * d), stream) != cudaSuccess) return 3;
    if (cudaMemsetAsync(counts, 0, sizeof(int64_t) * (size_t)kc, stream) != cudaSuccess) return 3;
    if (inertia && cudaMemsetAsync(inertia, 0, sizeof(double), stream) != cudaSuccess) return 3;
    return 0;
  }
  if (kc > 12288 || d > 1024) return 2;  // smem histogram / one thread per dimension
  size_t total = 0;
  KmWs w = carve(ws, n, d, kc, &total);
  const int nb = (int)((n + kKmBlockPts - 1) / kKmBlockPts);
  const int64_t gmax = n / kKmChunk + kc + 1;
  const size_t hs = sizeof(int32_t) * (size_t)kc;
  const int dt = (int)((d + 31) / 32 * 32);
  km_hist_kernel<<<nb, 256, hs, stream>>>(assign, n, kc, w.H, nb);
  km_scan_blk_kernel<<<(unsigned)kc, 256, 0, stream>>>(w.H, nb, w.cnt);
  km_scan_c_kernel<<<1, 1024, 0, stream>>>(w.cnt, kc, w.offsets, counts, w.chunk_base, w.chunk_j,
                                           w.n_chunks, w.done, sums, d, w.in_j);
  // W warps per scatter block, W per-warp histograms of kc counters in smem (<= 48 KiB)
  // (measured: the same 83 us at 4M points as one warp per block -- the per-block kc-sized
  // histogram work, not the serial walk, bounds it; a smem-staged coalesced copy-out was
  // slower)
  if (kc <= 1536)
    km_scatter_kernel<8><<<nb, 256, 8 * hs, stream>>>(assign, n, kc, w.H, nb, w.offsets, w.order);
  else if (kc <= 3072)
    km_scatter_kernel<4><<<nb, 128, 4 * hs, stream>>>(assign, n, kc, w.H, nb, w.offsets, w.order);
  else if (kc <= 6144)
    km_scatter_kernel<2><<<nb, 64, 2 * hs, stream>>>(assign, n, kc, w.H, nb, w.offsets, w.order);
  else
    km_scatter_kernel<1><<<nb, 32, hs, stream>>>(assign, n, kc, w.H, nb, w.offsets, w.order);
  int tpc_log2 = -1;  // float4 rows: d / 4 lanes per chunk, a power of two <= 32
  if (d % 4 == 0 && ldx % 4 == 0 && (reinterpret_cast<uintptr_t>(X) % 16) == 0 &&
      (reinterpret_cast<uintptr_t>(sums) % 16) == 0)
    for (int l = 0; l <= 5; l++)
      if ((int64_t)(4 << l) == d) tpc_log2 = l;
  if (tpc_log2 >= 0) {
    const unsigned blocks = (unsigned)((gmax + kKmVecChunks - 1) / kKmVecChunks);
    const unsigned threads = (unsigned)(kKmVecChunks << tpc_log2);
    if (inertia)
      km_chunk_vec_kernel<true><<<blocks, threads, 0, stream>>>(
          X, d, ldx, w.order, w.offsets, counts, w.chunk_base, w.chunk_j, w.n_chunks, best_key,
          w.part, w.part_in, w.done, sums, w.in_j, tpc_log2);
    else
      km_chunk_vec_kernel<false><<<blocks, threads, 0, stream>>>(
          X, d, ldx, w.order, w.offsets, counts, w.chunk_base, w.chunk_j, w.n_chunks, best_key,
          w.part, nullptr, w.done, sums, w.in_j, tpc_log2);
  } else {
    km_chunk_kernel<<<(unsigned)gmax, dt, 0, stream>>>(X, d, ldx, w.order, w.offsets, counts,
                                                       w.chunk_base, w.chunk_j, w.n_chunks, best_key,
                                                       w.part, inertia ? w.part_in : nullptr, w.done,
                                                       sums, w.in_j);
  }
  if (inertia) km_inertia_kernel<<<1, 1024, 0, stream>>>(w.in_j, kc, inertia);
  return cudaGetLastError() == cudaSuccess ? 0 : 3;
}

__global__ void kmeans_finalize_kernel(const double* __restrict__ sums,
                                       const int64_t* __restrict__ counts, int64_t kc, int64_t d,
                                       float* __restrict__ centroids) {
  const int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (e >= kc * d) return;
  const int64_t j = e / d;
  const int64_t c = counts[j];
  if (c > 0) centroids[e] = (float)__ddiv_rn(sums[e], (double)c);  // fp64 divide, one rounding
}

// The kMeans exchange step fused with the update (SURVEY 8e follow-up, the "fused NVLS /
// symmetric-memory reduction in the step's tail"): every rank reads the partial sums and
// counts of ALL ranks straight from their (peer-mapped, e.g. torch SymmetricMemory) buffers,
// adds them in rank order 0, 1, ..., P-1 -- the same fixed order on every rank, so the
// reduced sums and hence the centroids are bitwise identical across ranks without a
// collective library call -- writes the reduced sums / counts locally and finalizes.
// One thread per (j, t): reads P fp64 + P int64 over NVLink (P2P loads), no atomics.
struct PeerPtrs {
  const double* sums[kMaxPeers];
  const int64_t* counts[kMaxPeers];
};

__global__ void kmeans_peer_reduce_finalize_kernel(PeerPtrs pp, int nranks, int64_t kc, int64_t d,
                                                   double* __restrict__ sums_out,
                                                   int64_t* __restrict__ counts_out,
                                                   float* __restrict__ centroids) {
  const int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (e >= kc * d) return;
  const int64_t j = e / d, t = e - j * d;
  double s = 0.0;
  int64_t c = 0;
  for (int r = 0; r < nranks; r++) {  // fixed rank order: identical bits on every rank
    s = __dadd_rn(s, pp.sums[r][e]);
    c += pp.counts[r][j];
  }
  if (sums_out) sums_out[e] = s;
  if (counts_out && t == 0) counts_out[j] = c;
  if (c > 0) centroids[e] = (float)__ddiv_rn(s, (double)c);
}

int launch_kmeans_peer_reduce_finalize(const double* const* peer_sums,
                                       const int64_t* const* peer_counts, int nranks, int64_t kc,
                                       int64_t d, double* sums_out, int64_t* counts_out,
                                       float* centroids, cudaStream_t stream) {
  if (kc * d <= 0) return 0;
  PeerPtrs pp = {};
  for (int r = 0; r < nranks; r++) {
    pp.sums[r] = peer_sums[r];
    pp.counts[r] = peer_counts[r];
  }
  kmeans_peer_reduce_finalize_kernel<<<(unsigned)((kc * d + 255) / 256), 256, 0, stream>>>(
      pp, nranks, kc, d, sums_out, counts_out, centroids);
  return cudaGetLastError() == cudaSuccess ? 0 : 3;
}

int launch_kmeans_finalize(const double* sums, const int64_t* counts, int64_t kc, int64_t d,
                           float* centroids, cudaStream_t stream) {
  if (kc * d <= 0) return 0;
  kmeans_finalize_kernel<<<(unsigned)((kc * d + 255) / 256), 256, 0, stream>>>(sums, counts, kc, d,
                                                                                 centroids);
  return cudaGetLastError() == cudaSuccess ? 0 : 3;
}

}  // namespace egemm
