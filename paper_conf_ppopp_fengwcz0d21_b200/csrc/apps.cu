// apps.cu -- the CUDA-core kernels around the tensor-core kernel for the paper's two
// case studies (kNN [9] and kMeans [2]):
// fp64-accumulated row norms, the cross-slice kNN top-k merge, the kMeans centroid
// partial sums / counts / inertia and the centroid update, and D = C for K == 0.
#include <cuda_runtime.h>
#include <cstdint>
#include "egemm_internal.h"

namespace egemm {

// ||x_i||^2 accumulated in fp64, rounded once to fp32.  One warp per row.
__global__ void rownorm_kernel(const float* __restrict__ x, int64_t rows, int64_t d, int64_t ld,
                               float* __restrict__ out) {
  const int64_t warp = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int lane = threadIdx.x & 31;
  const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t r = warp; r < rows; r += nwarps) {
    const float* xr = x + r * ld;
    double s = 0.0;
    for (int64_t t = lane; t < d; t += 32) {
      double v = (double)xr[t];
      s = fma(v, v, s);
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
    if (lane == 0) out[r] = (float)s;
  }
}

int launch_rownorm(const float* x, int64_t rows, int64_t d, int64_t ld, float* out,
                   cudaStream_t stream) {
  if (rows <= 0) return 0;
  int64_t blocks = (rows * 32 + 255) / 256;
  int64_t cap = (int64_t)num_sms() * 8;
  if (blocks > cap) blocks = cap;
  rownorm_kernel<<<(unsigned)blocks, 256, 0, stream>>>(x, rows, d, ld, out);
  return cudaGetLastError() == cudaSuccess ? 0 : 3;
}

// Merge the per-slice sorted (key, idx) lists of each query into the final top-k,
// ascending by (key, idx); distance = max(0, ||q||^2 + key) (reading R11).
template <int KN>
__global__ void knn_merge_kernel(const float* __restrict__ pk, const int32_t* __restrict__ pi,
                                 int n_slices, int64_t nq, int k, const float* __restrict__ qnorm,
                                 int32_t* __restrict__ out_idx, float* __restrict__ out_dist) {
  const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= nq) return;
  float kd[KN];
  int ki[KN];
#pragma unroll
  for (int t = 0; t < KN; t++) { kd[t] = __int_as_float(0x7f800000); ki[t] = 0x7fffffff; }
  for (int s = 0; s < n_slices; s++) {
    const int64_t o = ((int64_t)s * nq + i) * k;
    for (int t = 0; t < k; t++) {
      float key = pk[o + t];
      int idx = pi[o + t];
      if (key < kd[KN - 1] || (key == kd[KN - 1] && idx < ki[KN - 1])) {
        kd[KN - 1] = key;
        ki[KN - 1] = idx;
#pragma unroll
        for (int u = KN - 1; u > 0; u--) {
          bool sw = (kd[u] < kd[u - 1]) || (kd[u] == kd[u - 1] && ki[u] < ki[u - 1]);
          float a = kd[u], b = kd[u - 1];
          int ia = ki[u], ib = ki[u - 1];
          kd[u] = sw ? b : a; kd[u - 1] = sw ? a : b;
          ki[u] = sw ? ib : ia; ki[u - 1] = sw ? ia : ib;
        }
      } else if (key > kd[KN - 1]) {
        break;  // each partial list is ascending
      }
    }
  }
  const float qn = qnorm[i];
#pragma unroll
  for (int t = 0; t < KN; t++) {
    if (t < k) {
      out_idx[i * k + t] = ki[t] == 0x7fffffff ? -1 : ki[t];
      float dd = __fadd_rn(qn, kd[t]);
      out_dist[i * k + t] = dd > 0.f ? dd : 0.f;
    }
  }
}

int launch_knn_merge(const float* part_key, const int32_t* part_idx, int n_slices, int64_t nq,
                     int k, const float* qnorm, int32_t* out_idx, float* out_dist,
                     cudaStream_t stream) {
  if (nq <= 0) return 0;
  unsigned blocks = (unsigned)((nq + 127) / 128);
  knn_merge_kernel<16><<<blocks, 128, 0, stream>>>(part_key, part_idx, n_slices, nq, k, qnorm,
                                                    out_idx, out_dist);
  return cudaGetLastError() == cudaSuccess ? 0 : 3;
}

// ---------------------------------------------------------------------------------
// kMeans partial sums, deterministic and in the oracle's order (reading R20):
//   sums[j][t] = sum over i ascending with a_i == j of (double)x_i[t]   (fp64, sequential)
//   counts[j]  = #{i : a_i == j};  inertia = sum_i ||x_i||^2 + best_key_i (fp64)
// Instead of 4M x 64 fp64 atomics, a stable counting sort groups the point indices by
// centroid (ascending i inside each group) and one thread per (centroid, dim) adds its
// group sequentially -- the same additions in the same order as the CPU oracle, so the
// sums are bitwise equal to it for equal assignments.
//   A: per-block histogram H[j][b]    B1: per-centroid scan over blocks   B2: scan over j
//   C: stable scatter (warp-serial chunks, match_any ranks)   D: sequential group sums
constexpr int kKmBlockPts = 4096;  // points per histogram / scatter block

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

// one block per centroid j: exclusive scan of H[j][0..nb) in place, count[j] = total
__global__ void km_scan_blocks_kernel(int32_t* __restrict__ H, int nb, int32_t* __restrict__ cnt) {
  __shared__ int32_t carry;
  __shared__ int32_t warp_tot[32];
  const int64_t j = blockIdx.x;
  int32_t* row = H + j * nb;
  if (threadIdx.x == 0) carry = 0;
  __syncthreads();
  for (int base = 0; base < nb; base += blockDim.x) {
    const int b = base + threadIdx.x;
    const int32_t v = b < nb ? row[b] : 0;
    int32_t x = v;  // inclusive warp scan
    for (int o = 1; o < 32; o <<= 1) {
      int32_t y = __shfl_up_sync(0xffffffffu, x, o);
      if ((threadIdx.x & 31) >= o) x += y;
    }
    if ((threadIdx.x & 31) == 31) warp_tot[threadIdx.x >> 5] = x;
    __syncthreads();
    int32_t wpre = 0;
    for (int w = 0; w < (int)(threadIdx.x >> 5); w++) wpre += warp_tot[w];
    const int32_t excl = carry + wpre + x - v;
    __syncthreads();
    if (b < nb) row[b] = excl;
    if (threadIdx.x == blockDim.x - 1) carry = excl + v;
    __syncthreads();
  }
  if (threadIdx.x == 0) cnt[j] = carry;
}

// single block of 1024 threads: offsets[j] = exclusive scan of cnt over j; counts = cnt
__global__ void km_scan_centroids_kernel(const int32_t* __restrict__ cnt, int64_t kc,
                                         int64_t* __restrict__ offsets, int64_t* __restrict__ counts) {
  __shared__ int64_t carry;
  __shared__ int64_t warp_tot[32];
  if (threadIdx.x == 0) carry = 0;
  __syncthreads();
  for (int64_t base = 0; base < kc; base += blockDim.x) {
    const int64_t j = base + threadIdx.x;
    const int64_t v = j < kc ? (int64_t)cnt[j] : 0;
    int64_t x = v;
    for (int o = 1; o < 32; o <<= 1) {
      int64_t y = __shfl_up_sync(0xffffffffu, x, o);
      if ((threadIdx.x & 31) >= o) x += y;
    }
    if ((threadIdx.x & 31) == 31) warp_tot[threadIdx.x >> 5] = x;
    __syncthreads();
    int64_t wpre = 0;
    for (int w = 0; w < (int)(threadIdx.x >> 5); w++) wpre += warp_tot[w];
    const int64_t excl = carry + wpre + x - v;
    __syncthreads();
    if (j < kc) { offsets[j] = excl; counts[j] = v; }
    if (threadIdx.x == blockDim.x - 1) carry = excl + v;
    __syncthreads();
  }
}

// one warp per block of kKmBlockPts points, chunks of 32 in order: stable placement
__global__ void km_scatter_kernel(const int32_t* __restrict__ assign, int64_t n, int64_t kc,
                                  const int32_t* __restrict__ H, int nb,
                                  const int64_t* __restrict__ offsets, int32_t* __restrict__ order) {
  extern __shared__ int32_t run[];
  const int lane = threadIdx.x;
  for (int64_t j = lane; j < kc; j += 32) run[j] = 0;
  __syncwarp();
  const int64_t i0 = (int64_t)blockIdx.x * kKmBlockPts;
  const int64_t i1 = min(n, i0 + kKmBlockPts);
  for (int64_t c = i0; c < i1; c += 32) {
    const int64_t i = c + lane;
    const bool valid = i < i1;
    const int a = valid ? assign[i] : -1 - lane;  // invalid lanes never match a real bucket
    const uint32_t peers = __match_any_sync(0xffffffffu, a);
    const int rank = __popc(peers & ((1u << lane) - 1u));
    if (valid) {
      const int64_t pos = offsets[a] + H[(int64_t)a * nb + blockIdx.x] + run[a] + rank;
      order[pos] = (int32_t)i;
    }
    __syncwarp();
    const int leader = __ffs(peers) - 1;
    if (valid && lane == leader) run[a] += __popc(peers);
    __syncwarp();
  }
}

// one block per centroid, one thread per dimension: sequential fp64 sums in ascending i.
// Rows are gathered 32 at a time (32 independent loads in flight per thread) and then
// added in order, so the dependent add chain never waits on memory for every row.
__global__ void km_segsum_kernel(const float* __restrict__ X, int64_t d, int64_t ldx,
                                 const int32_t* __restrict__ order,
                                 const int64_t* __restrict__ offsets,
                                 const int64_t* __restrict__ counts,
                                 const float* __restrict__ best_key, double* __restrict__ sums,
                                 double* __restrict__ inertia) {
  __shared__ int32_t sidx[32];
  const int64_t j = blockIdx.x;
  const int64_t p0 = offsets[j], cnt = counts[j];
  const int64_t t = threadIdx.x;
  const bool active = t < d;
  double s = 0.0, q = 0.0, bk = 0.0;
  for (int64_t base = 0; base < cnt; base += 32) {
    const int nrow = (int)min((int64_t)32, cnt - base);
    __syncthreads();
    if (threadIdx.x < 32) sidx[threadIdx.x] = threadIdx.x < nrow ? order[p0 + base + threadIdx.x] : 0;
    __syncthreads();
    float xv[32];
#pragma unroll
    for (int r = 0; r < 32; r++)
      xv[r] = (active && r < nrow) ? __ldg(X + (int64_t)sidx[r] * ldx + t) : 0.f;
#pragma unroll
    for (int r = 0; r < 32; r++) {
      if (r < nrow) {
        s = __dadd_rn(s, (double)xv[r]);
        q = fma((double)xv[r], (double)xv[r], q);
      }
    }
    if (inertia && threadIdx.x == 0)
      for (int r = 0; r < nrow; r++) bk += (double)best_key[sidx[r]];
  }
  if (active) sums[j * d + t] = s;
  if (inertia) {
    if (active) atomicAdd(inertia, q);
    if (threadIdx.x == 0) atomicAdd(inertia, bk);
  }
}

size_t kmeans_accumulate_ws(int64_t n, int64_t kc) {
  const int64_t nb = (n + kKmBlockPts - 1) / kKmBlockPts;
  auto al = [](size_t x) { return (x + 255) & ~size_t(255); };
  return al(sizeof(int32_t) * (size_t)(kc * (nb > 0 ? nb : 1))) + al(sizeof(int32_t) * (size_t)kc) +
         al(sizeof(int64_t) * (size_t)kc) + al(sizeof(int32_t) * (size_t)(n > 0 ? n : 1));
}

int launch_kmeans_accumulate(const float* X, int64_t n, int64_t d, int64_t ldx,
                             const int32_t* assign, const float* best_key, int64_t kc, double* sums,
                             int64_t* counts, double* inertia, void* ws, cudaStream_t stream) {
  if (inertia && cudaMemsetAsync(inertia, 0, sizeof(double), stream) != cudaSuccess) return 3;
  if (n <= 0) {
    if (cudaMemsetAsync(sums, 0, sizeof(double) * (size_t)(kc * d), stream) != cudaSuccess) return 3;
    if (cudaMemsetAsync(counts, 0, sizeof(int64_t) * (size_t)kc, stream) != cudaSuccess) return 3;
    return 0;
  }
  if (kc > 12288) return 2;  // smem histogram / run counters
  const int nb = (int)((n + kKmBlockPts - 1) / kKmBlockPts);
  auto al = [](size_t x) { return (x + 255) & ~size_t(255); };
  char* w = reinterpret_cast<char*>(ws);
  int32_t* H = reinterpret_cast<int32_t*>(w);
  w += al(sizeof(int32_t) * (size_t)(kc * nb));
  int32_t* cnt = reinterpret_cast<int32_t*>(w);
  w += al(sizeof(int32_t) * (size_t)kc);
  int64_t* offsets = reinterpret_cast<int64_t*>(w);
  w += al(sizeof(int64_t) * (size_t)kc);
  int32_t* order = reinterpret_cast<int32_t*>(w);
  const size_t hs = sizeof(int32_t) * (size_t)kc;
  km_hist_kernel<<<nb, 256, hs, stream>>>(assign, n, kc, H, nb);
  km_scan_blocks_kernel<<<(unsigned)kc, 256, 0, stream>>>(H, nb, cnt);
  km_scan_centroids_kernel<<<1, 1024, 0, stream>>>(cnt, kc, offsets, counts);
  km_scatter_kernel<<<nb, 32, hs, stream>>>(assign, n, kc, H, nb, offsets, order);
  const int threads = d >= 1024 ? 1024 : (int)((d + 31) / 32 * 32);
  km_segsum_kernel<<<(unsigned)kc, threads, 0, stream>>>(X, d, ldx, order, offsets, counts,
                                                          best_key, sums, inertia);
  return cudaGetLastError() == cudaSuccess ? 0 : 3;
}

__global__ void kmeans_finalize_kernel(const double* __restrict__ sums,
                                       const int64_t* __restrict__ counts, int64_t kc, int64_t d,
                                       float* __restrict__ centroids) {
  const int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (e >= kc * d) return;
  const int64_t j = e / d;
  const int64_t c = counts[j];
  if (c > 0) centroids[e] = (float)(sums[e] / (double)c);  // fp64 divide, one rounding
}

int launch_kmeans_finalize(const double* sums, const int64_t* counts, int64_t kc, int64_t d,
                           float* centroids, cudaStream_t stream) {
  if (kc * d <= 0) return 0;
  kmeans_finalize_kernel<<<(unsigned)((kc * d + 255) / 256), 256, 0, stream>>>(sums, counts, kc, d,
                                                                                 centroids);
  return cudaGetLastError() == cudaSuccess ? 0 : 3;
}

__global__ void fill_c_kernel(int64_t M, int64_t N, const float* __restrict__ C, int64_t ldc,
                              float* __restrict__ D, int64_t ldd) {
  const int64_t total = M * N;
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < total; e += stride) {
    int64_t i = e / N, j = e - i * N;
    D[i * ldd + j] = C ? C[i * ldc + j] : 0.f;
  }
}

int launch_fill_c(int64_t M, int64_t N, const float* C, int64_t ldc, float* D, int64_t ldd,
                  cudaStream_t stream) {
  if (M <= 0 || N <= 0) return 0;
  int64_t blocks = (M * N + 255) / 256;
  int64_t cap = (int64_t)num_sms() * 8;
  if (blocks > cap) blocks = cap;
  fill_c_kernel<<<(unsigned)blocks, 256, 0, stream>>>(M, N, C, ldc, D, ldd);
  return cudaGetLastError() == cudaSuccess ? 0 : 3;
}

}  // namespace egemm
