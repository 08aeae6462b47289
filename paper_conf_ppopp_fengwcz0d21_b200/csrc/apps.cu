// apps.cu -- the CUDA-core kernels around the tensor-core kernel for the paper's two
// case studies (kNN [9] and kMeans [2]):
// fp64-accumulated row norms, the cross-slice kNN top-k merge, and D = C for K == 0
// (the kMeans sums and update live in kmeans.cu).
#include <cuda_runtime.h>
#include <cstdint>
#include "egemm_internal.h"

namespace egemm {

// ||x_i||^2 = sum_t x_it^2 accumulated in fp64 in ascending t (every square is exact in
// fp64), rounded once to fp32 -- the plain definition (reading R22), so the norms are
// bitwise reproducible by a sequential loop.  One thread per row: a warp's 32 rows are
// staged through shared memory in 32-column slabs (coalesced 128-B row segments), then each
// lane adds its own row's slab in order.
constexpr int kNormSlab = 32;
__global__ void __launch_bounds__(256) rownorm_kernel(const float* __restrict__ x, int64_t rows,
                                                      int64_t d, int64_t ld, float* __restrict__ out) {
  __shared__ float slab[8][32][kNormSlab + 1];
  const int w = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int64_t nwarps = (int64_t)gridDim.x * 8;
  for (int64_t r0 = ((int64_t)blockIdx.x * 8 + w) * 32; r0 < rows; r0 += nwarps * 32) {
    double s = 0.0;
    for (int64_t t0 = 0; t0 < d; t0 += kNormSlab) {
      __syncwarp();
#pragma unroll
      for (int rr = 0; rr < 32; rr++) {  // row r0 + rr, columns t0 + lane (all 32 loads in flight)
        const int64_t r = r0 + rr, t = t0 + lane;
        slab[w][rr][lane] = (r < rows && t < d) ? __ldg(x + r * ld + t) : 0.f;
      }
      __syncwarp();
      const int tn = (d - t0 < kNormSlab) ? (int)(d - t0) : kNormSlab;
      for (int t = 0; t < tn; t++) {
        const double v = (double)slab[w][lane][t];
        s = __dadd_rn(s, __dmul_rn(v, v));  // exact square, one rounding per add
      }
    }
    if (r0 + lane < rows) out[r0 + lane] = __double2float_rn(s);
  }
}

int launch_rownorm(const float* x, int64_t rows, int64_t d, int64_t ld, float* out,
                   cudaStream_t stream) {
  if (rows <= 0) return 0;
  int64_t blocks = (rows + 255) / 256;  // 8 warps x 32 rows per block and round
  int64_t cap = (int64_t)num_sms() * 8;
  if (blocks > cap) blocks = cap;
  rownorm_kernel<<<(unsigned)blocks, 256, 0, stream>>>(x, rows, d, ld, out);
  return cudaGetLastError() == cudaSuccess ? 0 : 3;
}

// Merge of n_lists sorted (key, idx) lists per query into the top k (reading R11 order:
// ascending key, ties by lower idx).  One warp per query.  Every valid entry's final rank is
// counted exactly -- its position in its own list plus, for every other list, the number
// of entries that precede it (a binary search; indices are distinct across lists, so no
// two valid entries compare equal) -- and the entries with rank < k are written there.
// Empty slots (idx < 0 or INT32_MAX) rank after everything and are never written; output
// slots beyond the number of valid entries get (-1, +inf).
__device__ __forceinline__ bool knn_before(float ka, int ia, float kb, int ib) {
  return ka < kb || (ka == kb && ia < ib);
}
__device__ __forceinline__ bool knn_valid(int i) { return i >= 0 && i != 0x7fffffff; }

__global__ void __launch_bounds__(256) knn_merge_kernel(const float* __restrict__ pk,
                                                        const int32_t* __restrict__ pi, int n_lists,
                                                        int64_t nq, int k_in, int k,
                                                        const float* __restrict__ qnorm,
                                                        int32_t* __restrict__ out_idx,
                                                        float* __restrict__ out_key) {
  const int lane = threadIdx.x & 31;
  const int64_t q = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  if (q >= nq) return;
  const float qn = qnorm ? qnorm[q] : 0.f;
  const int total = n_lists * k_in;
  int nvalid = 0;
  for (int c = lane; c < total; c += 32) {
    const int l = c / k_in, p = c - l * k_in;
    const int64_t o = ((int64_t)l * nq + q) * k_in;
    const int idx = pi[o + p];
    if (!knn_valid(idx)) continue;
    nvalid++;
    const float key = pk[o + p];
    int rank = p;  // entries of its own list before it (the list is sorted)
    for (int m = 0; m < n_lists && rank < k; m++) {
      if (m == l) continue;
      const int64_t om = ((int64_t)m * nq + q) * k_in;
      int lo = 0, hi = k_in;  // first position whose entry does not precede (key, idx)
      while (lo < hi) {
        const int mid = (lo + hi) >> 1;
        const int im = pi[om + mid];
        const bool before = knn_valid(im) && knn_before(pk[om + mid], im, key, idx);
        if (before) lo = mid + 1; else hi = mid;
      }
      rank += lo;
    }
    if (rank < k) {
      out_idx[q * k + rank] = idx;
      const float v = qnorm ? __fadd_rn(qn, key) : key;
      out_key[q * k + rank] = qnorm ? (v > 0.f ? v : 0.f) : v;
    }
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) nvalid += __shfl_xor_sync(0xffffffffu, nvalid, o);
  for (int t = nvalid + lane; t < k; t += 32) {
    out_idx[q * k + t] = -1;
    out_key[q * k + t] = __int_as_float(0x7f800000);
  }
}

int launch_knn_merge(const float* part_key, const int32_t* part_idx, int n_lists, int64_t nq,
                     int k_in, int k, const float* qnorm, int32_t* out_idx, float* out_key,
                     cudaStream_t stream) {
  if (nq <= 0) return 0;
  const int64_t blocks = (nq * 32 + 255) / 256;  // 8 queries per block
  knn_merge_kernel<<<(unsigned)blocks, 256, 0, stream>>>(part_key, part_idx, n_lists, nq, k_in, k,
                                                          qnorm, out_idx, out_key);
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
