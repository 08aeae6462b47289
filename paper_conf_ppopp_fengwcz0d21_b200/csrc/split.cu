// split.cu -- round-split of fp32 operands into fp16 hi / lo parts on the CUDA cores.
//
// Alg. 1 lines 2-3, Fig. 4b round-split:
//   hi = fp16_RN(x);   lo = fp16_RN(x - (float)hi)      (x - hi is exact in fp32)
// Rounding is cvt.rn (ties to even, reading R1 in DESIGN.md).  No -ftz / fast-math: fp32
// subnormals and fp16 subnormal lo parts are kept.
//
// HBM-bound: 4 B read + 4 B written per element.  Kernels use 128-bit loads/stores and a
// grid of 148 x (resident CTAs) for the contiguous case; the transposing variant (B stored
// K x N -> K-major N x K hi/lo) stages 64 x 64 tiles through shared memory.
#include <cuda_fp16.h>
#include <cstdint>
#include "egemm_internal.h"

namespace egemm {

struct SplitPair {
  uint32_t hi, lo;  // two packed fp16 each
};

__device__ __forceinline__ SplitPair split2(float a, float b, uint32_t& flags) {
  __half2 h = __floats2half2_rn(a, b);                 // cvt.rn.f16x2.f32
  float2 hf = __half22float2(h);
  __half2 l = __floats2half2_rn(a - hf.x, b - hf.y);  // residuals exact in fp32
  float aa = fabsf(a), ab = fabsf(b);
  // bit0: |x| >= 65520 (rounds to inf) or non-finite; bit1: 0 < |x| < 2^-3 (below 21-bit zone)
  flags |= (!(aa < 65520.f) || !(ab < 65520.f)) ? 1u : 0u;
  flags |= ((aa > 0.f && aa < 0.125f) || (ab > 0.f && ab < 0.125f)) ? 2u : 0u;
  SplitPair p;
  p.hi = *reinterpret_cast<uint32_t*>(&h);
  p.lo = *reinterpret_cast<uint32_t*>(&l);
  return p;
}

__device__ __forceinline__ void flush_flags(uint32_t flags, uint32_t* range_flags) {
  if (range_flags == nullptr) return;
  uint32_t any = __reduce_or_sync(0xffffffffu, flags);
  if (any && (threadIdx.x & 31) == 0) atomicOr(range_flags, any);
}

// Contiguous: x, hi, lo dense, n % 8 == 0 handled by the vector body, tail by scalars.
__global__ void __launch_bounds__(256) split_flat_kernel(const float* __restrict__ x, int64_t n,
                                                          uint16_t* __restrict__ hi,
                                                          uint16_t* __restrict__ lo,
                                                          uint32_t* range_flags) {
  uint32_t flags = 0;
  const int64_t nv = n >> 3;  // groups of 8 elements: 2 x 16 B in, 16 B + 16 B out
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  for (int64_t g = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; g < nv; g += stride) {
    const float4* src = reinterpret_cast<const float4*>(x) + 2 * g;
    float4 a = __ldcs(src);
    float4 b = __ldcs(src + 1);
    SplitPair p0 = split2(a.x, a.y, flags), p1 = split2(a.z, a.w, flags);
    SplitPair p2 = split2(b.x, b.y, flags), p3 = split2(b.z, b.w, flags);
    uint4 vh = make_uint4(p0.hi, p1.hi, p2.hi, p3.hi);
    uint4 vl = make_uint4(p0.lo, p1.lo, p2.lo, p3.lo);
    __stcs(reinterpret_cast<uint4*>(hi) + g, vh);
    __stcs(reinterpret_cast<uint4*>(lo) + g, vl);
  }
  // scalar tail (n % 8 elements), handled by the first threads of block 0
  if (blockIdx.x == 0) {
    int64_t t = (nv << 3) + threadIdx.x;
    if (t < n) {
      SplitPair p = split2(x[t], 0.f, flags);
      hi[t] = (uint16_t)(p.hi & 0xffffu);
      lo[t] = (uint16_t)(p.lo & 0xffffu);
    }
  }
  flush_flags(flags, range_flags);
}

// Strided, same orientation: one thread per element pair along cols.
__global__ void __launch_bounds__(256) split_strided_kernel(const float* __restrict__ x,
                                                             int64_t rows, int64_t cols,
                                                             int64_t ldx, uint16_t* __restrict__ hi,
                                                             uint16_t* __restrict__ lo,
                                                             int64_t ldo, uint32_t* range_flags) {
  uint32_t flags = 0;
  const int64_t total = rows * cols;
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < total; e += stride) {
    int64_t r = e / cols, c = e - r * cols;
    SplitPair p = split2(x[r * ldx + c], 0.f, flags);
    hi[r * ldo + c] = (uint16_t)(p.hi & 0xffffu);
    lo[r * ldo + c] = (uint16_t)(p.lo & 0xffffu);
  }
  flush_flags(flags, range_flags);
}

// Transposing: x is rows x cols (ldx); hi/lo are cols x rows (ldo).  64x64 tiles.
__global__ void __launch_bounds__(256) split_transpose_kernel(const float* __restrict__ x,
                                                               int64_t rows, int64_t cols,
                                                               int64_t ldx,
                                                               uint16_t* __restrict__ hi,
                                                               uint16_t* __restrict__ lo,
                                                               int64_t ldo, uint32_t* range_flags) {
  __shared__ uint32_t th[64][33];  // packed (hi,lo) of tile element [c][r] pairs
  __shared__ uint32_t tl[64][33];
  uint32_t flags = 0;
  const int64_t r0 = (int64_t)blockIdx.y * 64, c0 = (int64_t)blockIdx.x * 64;
  const int tx = threadIdx.x & 31, ty = threadIdx.x >> 5;  // 32 x 8
  // load: each thread reads x[r0 + ty + 8i][c0 + 2tx, 2tx+1]
  for (int i = 0; i < 8; i++) {
    int r = ty + 8 * i;
    int64_t gr = r0 + r, gc = c0 + 2 * tx;
    float a = 0.f, b = 0.f;
    if (gr < rows) {
      if (gc < cols) a = x[gr * ldx + gc];
      if (gc + 1 < cols) b = x[gr * ldx + gc + 1];
    }
    SplitPair p = split2(a, b, flags);
    // element (r, 2tx) and (r, 2tx+1); store column-major for the transposed write
    reinterpret_cast<uint16_t*>(&th[2 * tx][0])[r] = (uint16_t)(p.hi & 0xffffu);
    reinterpret_cast<uint16_t*>(&th[2 * tx + 1][0])[r] = (uint16_t)(p.hi >> 16);
    reinterpret_cast<uint16_t*>(&tl[2 * tx][0])[r] = (uint16_t)(p.lo & 0xffffu);
    reinterpret_cast<uint16_t*>(&tl[2 * tx + 1][0])[r] = (uint16_t)(p.lo >> 16);
  }
  __syncthreads();
  // write: output row = column c of x; each thread writes 2 consecutive fp16 (rows 2tx, 2tx+1)
  for (int i = 0; i < 8; i++) {
    int c = ty + 8 * i;
    int64_t oc = c0 + c;
    int64_t orow = r0 + 2 * tx;
    if (oc >= cols) continue;
    uint32_t vh = th[c][tx], vl = tl[c][tx];
    if (orow + 1 < rows && ((ldo & 1) == 0)) {
      *reinterpret_cast<uint32_t*>(hi + oc * ldo + orow) = vh;
      *reinterpret_cast<uint32_t*>(lo + oc * ldo + orow) = vl;
    } else {
      if (orow < rows) {
        hi[oc * ldo + orow] = (uint16_t)(vh & 0xffffu);
        lo[oc * ldo + orow] = (uint16_t)(vl & 0xffffu);
      }
      if (orow + 1 < rows) {
        hi[oc * ldo + orow + 1] = (uint16_t)(vh >> 16);
        lo[oc * ldo + orow + 1] = (uint16_t)(vl >> 16);
      }
    }
  }
  // padding elements contribute no flags (they are 0)
  flush_flags(flags, range_flags);
}

int launch_split(const float* x, int64_t rows, int64_t cols, int64_t ldx, uint16_t* hi,
                 uint16_t* lo, int64_t ldo, int transpose, uint32_t* range_flags,
                 cudaStream_t stream) {
  if (rows == 0 || cols == 0) return 0;
  int nsm = num_sms();
  if (!transpose) {
    bool flat = (ldx == cols && ldo == cols && ((uintptr_t)x % 16 == 0) &&
                 ((uintptr_t)hi % 16 == 0) && ((uintptr_t)lo % 16 == 0));
    if (flat) {
      int64_t n = rows * cols;
      int64_t groups = (n >> 3);
      int64_t blocks = (groups + 255) / 256;
      int64_t cap = (int64_t)nsm * 8;  // 8 x 256 threads resident per SM
      if (blocks > cap) blocks = cap;
      if (blocks < 1) blocks = 1;
      split_flat_kernel<<<(unsigned)blocks, 256, 0, stream>>>(x, n, hi, lo, range_flags);
    } else {
      int64_t n = rows * cols;
      int64_t blocks = (n + 255) / 256;
      int64_t cap = (int64_t)nsm * 8;
      if (blocks > cap) blocks = cap;
      split_strided_kernel<<<(unsigned)blocks, 256, 0, stream>>>(x, rows, cols, ldx, hi, lo, ldo,
                                                                  range_flags);
    }
  } else {
    dim3 grid((unsigned)((cols + 63) / 64), (unsigned)((rows + 63) / 64));
    split_transpose_kernel<<<grid, 256, 0, stream>>>(x, rows, cols, ldx, hi, lo, ldo, range_flags);
  }
  return cudaGetLastError() == cudaSuccess ? 0 : -1;
}

}  // namespace egemm
