// split.cu -- splitting fp32 operands into fp16 hi / lo parts on the CUDA cores.
//
// Round-split (MODE 0): Alg. 1 lines 2-3, Fig. 4b (P:759-771,
// P:826-856):  hi = fp16_RN(x);  lo = fp16_RN(x - (float)hi)   (x - hi exact in fp32).
// Rounding is cvt.rn (ties to even, reading R1 in DESIGN.md).
// Truncate-split (MODE 1, the Markidis variant the paper compares against, Fig. 4a,
// P:812-824; NEXT-1):  hi = fp16_RZ(x);  lo = fp16_RZ(x - (float)hi).
// No -ftz / fast-math: fp32 subnormals and fp16 subnormal lo parts are kept.
//
// HBM-bound: 4 B read + 4 B written per element.  The contiguous kernel moves 16 elements
// per thread and iteration (4 x 16-B loads, 2 x 16-B stores per output) on a grid of
// 148 x 8 CTAs; the transposing kernel (B stored K x N -> K-major N x K hi / lo) stages
// 128 x 64 tiles through shared memory and writes 16-B rows.
#include <cuda_fp16.h>
#include <cstdint>
#include "egemm_internal.h"

namespace egemm {

struct SplitPair {
  uint32_t hi, lo;  // two packed fp16 each (element a in the low half)
};

template <int MODE>
__device__ __forceinline__ SplitPair split2(float a, float b, uint32_t& flags) {
  uint32_t h, l;
  if (MODE == 0) asm("cvt.rn.f16x2.f32 %0, %1, %2;" : "=r"(h) : "f"(b), "f"(a));
  else asm("cvt.rz.f16x2.f32 %0, %1, %2;" : "=r"(h) : "f"(b), "f"(a));
  const __half2 hh = *reinterpret_cast<const __half2*>(&h);
  const float2 hf = __half22float2(hh);
  const float ra = __fsub_rn(a, hf.x), rb = __fsub_rn(b, hf.y);  // exact in fp32
  if (MODE == 0) asm("cvt.rn.f16x2.f32 %0, %1, %2;" : "=r"(l) : "f"(rb), "f"(ra));
  else asm("cvt.rz.f16x2.f32 %0, %1, %2;" : "=r"(l) : "f"(rb), "f"(ra));
  const float aa = fabsf(a), ab = fabsf(b);
  // bit0: |x| >= 65520 (rounds to inf) or non-finite; bit1: 0 < |x| < 2^-3 (below 21-bit zone)
  flags |= (!(aa < 65520.f) || !(ab < 65520.f)) ? 1u : 0u;
  flags |= ((aa > 0.f && aa < 0.125f) || (ab > 0.f && ab < 0.125f)) ? 2u : 0u;
  return SplitPair{h, l};
}

__device__ __forceinline__ void flush_flags(uint32_t flags, uint32_t* range_flags) {
  if (range_flags == nullptr) return;
  uint32_t any = __reduce_or_sync(0xffffffffu, flags);
  if (any && (threadIdx.x & 31) == 0) atomicOr(range_flags, any);
}

// Contiguous x, hi, lo: 16 elements per thread-iteration, scalar tail.
template <int MODE>
__global__ void __launch_bounds__(256) split_flat_kernel(const float* __restrict__ x, int64_t n,
                                                          uint16_t* __restrict__ hi,
                                                          uint16_t* __restrict__ lo,
                                                          uint32_t* range_flags) {
  uint32_t flags = 0;
  const int64_t nv = n >> 4;
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  for (int64_t g = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; g < nv; g += stride) {
    const float4* src = reinterpret_cast<const float4*>(x) + 4 * g;
    float4 v[4];
#pragma unroll
    for (int i = 0; i < 4; i++) v[i] = __ldcs(src + i);
    uint32_t h[8], l[8];
#pragma unroll
    for (int i = 0; i < 4; i++) {
      SplitPair p0 = split2<MODE>(v[i].x, v[i].y, flags), p1 = split2<MODE>(v[i].z, v[i].w, flags);
      h[2 * i] = p0.hi; h[2 * i + 1] = p1.hi;
      l[2 * i] = p0.lo; l[2 * i + 1] = p1.lo;
    }
    uint4* dh = reinterpret_cast<uint4*>(hi) + 2 * g;
    uint4* dl = reinterpret_cast<uint4*>(lo) + 2 * g;
    __stcs(dh, make_uint4(h[0], h[1], h[2], h[3]));
    __stcs(dh + 1, make_uint4(h[4], h[5], h[6], h[7]));
    __stcs(dl, make_uint4(l[0], l[1], l[2], l[3]));
    __stcs(dl + 1, make_uint4(l[4], l[5], l[6], l[7]));
  }
  if (blockIdx.x == 0) {  // scalar tail (n % 16 elements)
    const int64_t t = (nv << 4) + threadIdx.x;
    if (t < n) {
      SplitPair p = split2<MODE>(x[t], 0.f, flags);
      hi[t] = (uint16_t)(p.hi & 0xffffu);
      lo[t] = (uint16_t)(p.lo & 0xffffu);
    }
  }
  flush_flags(flags, range_flags);
}

// Strided, same orientation: one thread per element.
template <int MODE>
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
    SplitPair p = split2<MODE>(x[r * ldx + c], 0.f, flags);
    hi[r * ldo + c] = (uint16_t)(p.hi & 0xffffu);
    lo[r * ldo + c] = (uint16_t)(p.lo & 0xffffu);
  }
  flush_flags(flags, range_flags);
}

// Transposing: x is rows x cols (ldx); hi/lo are cols x rows (ldo).  Tiles of 128 x-rows
// x 64 x-cols: coalesced 8-B loads along x's rows, split, transposed into shared memory,
// then each output row segment (128 fp16 = 256 B) written as 16-B vectors.
constexpr int kTR = 128, kTC = 64, kTP = kTR + 8;  // pitch keeps 16-B row alignment

template <int MODE>
__global__ void __launch_bounds__(256) split_transpose_kernel(const float* __restrict__ x,
                                                               int64_t rows, int64_t cols,
                                                               int64_t ldx,
                                                               uint16_t* __restrict__ hi,
                                                               uint16_t* __restrict__ lo,
                                                               int64_t ldo, uint32_t* range_flags) {
  __shared__ __align__(16) uint16_t th[kTC][kTP];
  __shared__ __align__(16) uint16_t tl[kTC][kTP];
  uint32_t flags = 0;
  const int64_t r0 = (int64_t)blockIdx.y * kTR, c0 = (int64_t)blockIdx.x * kTC;
  const int tx = threadIdx.x & 31, ty = threadIdx.x >> 5;  // 32 x 8
  const bool vec_in = ((ldx & 1) == 0) && ((reinterpret_cast<uintptr_t>(x) & 7) == 0);
  const int64_t gc = c0 + 2 * tx;
#pragma unroll 4
  for (int i = 0; i < kTR / 8; i++) {
    const int r = ty + 8 * i;
    const int64_t gr = r0 + r;
    float a = 0.f, b = 0.f;
    if (gr < rows) {
      const float* src = x + gr * ldx + gc;
      if (vec_in && gc + 1 < cols) {
        const float2 t = __ldcs(reinterpret_cast<const float2*>(src));
        a = t.x;
        b = t.y;
      } else {
        if (gc < cols) a = src[0];
        if (gc + 1 < cols) b = src[1];
      }
    }
    SplitPair p = split2<MODE>(a, b, flags);
    th[2 * tx][r] = (uint16_t)(p.hi & 0xffffu);
    th[2 * tx + 1][r] = (uint16_t)(p.hi >> 16);
    tl[2 * tx][r] = (uint16_t)(p.lo & 0xffffu);
    tl[2 * tx + 1][r] = (uint16_t)(p.lo >> 16);
  }
  __syncthreads();
  // output rows oc = c0 + c (64 of them), 128 fp16 each = 16 chunks of 8: 4 per thread
  const bool vec_out = ((ldo & 7) == 0) && ((reinterpret_cast<uintptr_t>(hi) & 15) == 0) &&
                       ((reinterpret_cast<uintptr_t>(lo) & 15) == 0);
#pragma unroll
  for (int i = 0; i < 4; i++) {
    const int idx = threadIdx.x + 256 * i;  // 0 .. 1023
    const int c = idx >> 4, ch = idx & 15;
    const int64_t oc = c0 + c, orow = r0 + ch * 8;
    if (oc >= cols || orow >= rows) continue;
    if (vec_out && orow + 8 <= rows) {
      *reinterpret_cast<uint4*>(hi + oc * ldo + orow) = *reinterpret_cast<const uint4*>(&th[c][ch * 8]);
      *reinterpret_cast<uint4*>(lo + oc * ldo + orow) = *reinterpret_cast<const uint4*>(&tl[c][ch * 8]);
    } else {
      for (int e = 0; e < 8 && orow + e < rows; e++) {
        hi[oc * ldo + orow + e] = th[c][ch * 8 + e];
        lo[oc * ldo + orow + e] = tl[c][ch * 8 + e];
      }
    }
  }
  flush_flags(flags, range_flags);  // padding elements are 0: they raise no flag
}

template <int MODE>
static void launch_mode(const float* x, int64_t rows, int64_t cols, int64_t ldx, uint16_t* hi,
                        uint16_t* lo, int64_t ldo, int transpose, uint32_t* range_flags,
                        cudaStream_t stream) {
  const int nsm = num_sms();
  if (!transpose) {
    const bool flat = (ldx == cols && ldo == cols && ((uintptr_t)x % 16 == 0) &&
                       ((uintptr_t)hi % 16 == 0) && ((uintptr_t)lo % 16 == 0));
    const int64_t n = rows * cols;
    if (flat) {
      int64_t blocks = ((n >> 4) + 255) / 256;
      const int64_t cap = (int64_t)nsm * 8;  // 8 x 256 threads resident per SM
      if (blocks > cap) blocks = cap;
      if (blocks < 1) blocks = 1;
      split_flat_kernel<MODE><<<(unsigned)blocks, 256, 0, stream>>>(x, n, hi, lo, range_flags);
    } else {
      int64_t blocks = (n + 255) / 256;
      const int64_t cap = (int64_t)nsm * 8;
      if (blocks > cap) blocks = cap;
      split_strided_kernel<MODE><<<(unsigned)blocks, 256, 0, stream>>>(x, rows, cols, ldx, hi, lo,
                                                                        ldo, range_flags);
    }
  } else {
    dim3 grid((unsigned)((cols + kTC - 1) / kTC), (unsigned)((rows + kTR - 1) / kTR));
    split_transpose_kernel<MODE><<<grid, 256, 0, stream>>>(x, rows, cols, ldx, hi, lo, ldo,
                                                           range_flags);
  }
}

int launch_split(const float* x, int64_t rows, int64_t cols, int64_t ldx, uint16_t* hi,
                 uint16_t* lo, int64_t ldo, int transpose, uint32_t* range_flags,
                 cudaStream_t stream, int mode) {
  if (rows == 0 || cols == 0) return 0;
  if (mode == 1) launch_mode<1>(x, rows, cols, ldx, hi, lo, ldo, transpose, range_flags, stream);
  else launch_mode<0>(x, rows, cols, ldx, hi, lo, ldo, transpose, range_flags, stream);
  return cudaGetLastError() == cudaSuccess ? 0 : -1;
}

}  // namespace egemm
