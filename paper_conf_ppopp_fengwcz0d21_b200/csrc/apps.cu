// apps.cu -- the CUDA-core kernels around the tensor-core kernel for the paper's two
// case studies (kNN [9] and kMeans [2]):
// fp64-accumulated row norms, the cross-slice kNN top-k merge, and D = C for K == 0
// (the kMeans sums and update live in kmeans.cu).
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
