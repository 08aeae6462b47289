// split.cu -- splitting fp32 operands into fp16 hi / lo parts on the CUDA cores.
//
// Round-split (MODE 0): Alg. 1 lines 2-3, Fig. 4b (P:759-771,
// P:826-856):  hi = fp16_RN(x);  lo = fp16_RN(x - (float)hi)   (x - hi exact in fp32).
// Rounding is cvt.rn (ties to even, reading R1 in DESIGN.md).
// Truncate-split (MODE 1, the Markidis variant the paper compares against, Fig. 4a,
// P:812-824; NEXT-1):  hi = fp16_RZ(x);  lo = fp16_RZ(x - (float)hi).
// No -ftz / fast-math: fp32 subnormals and fp16 subnormal lo parts are kept.
//
// HBM-bound: 4 B read + 4 B written per element.  The contiguous kernel moves 8 elements
// per thread and iteration (2 x 16-B loads, one 16-B store per output) on a grid of
// 148 x 8 CTAs; the transposing kernel (B stored K x N -> K-major N x K hi / lo) stages
// 64 x 64 tiles through shared memory, splitting row pairs so the transpose moves packed
// fp16x2 words and writes 16 B per store.  The range-flag tests are compiled out unless
// the caller passes range_flags.  (Measured: wider 16-element flat iterations were slower.)
#include <cuda_fp16.h>
#include <cstdint>
#include "egemm_internal.h"
#include "ptx.cuh"

namespace egemm {

struct SplitPair {
  uint32_t hi, lo;  // two packed fp16 each (element a in the low half)
};

template <int MODE, bool FLAGS = true>
__device__ __forceinline__ SplitPair split2(float a, float b, uint32_t& flags) {
  uint32_t h, l;
  if constexpr (MODE == 2) {  // bf16 parts (NEXT-3): a bf16 is the top half of an fp32 pattern
    asm("cvt.rn.bf16x2.f32 %0, %1, %2;" : "=r"(h) : "f"(b), "f"(a));
    const float ra = __fsub_rn(a, __uint_as_float(h << 16));
    const float rb = __fsub_rn(b, __uint_as_float(h & 0xffff0000u));  // exact in fp32
    asm("cvt.rn.bf16x2.f32 %0, %1, %2;" : "=r"(l) : "f"(rb), "f"(ra));
    return SplitPair{h, l};
  }
  if (MODE == 0) asm("cvt.rn.f16x2.f32 %0, %1, %2;" : "=r"(h) : "f"(b), "f"(a));
  else asm("cvt.rz.f16x2.f32 %0, %1, %2;" : "=r"(h) : "f"(b), "f"(a));
  float ra, rb;
  ptx::residual2(h, a, b, ra, rb);  // x - hi, exact in fp32
  if (MODE == 0) asm("cvt.rn.f16x2.f32 %0, %1, %2;" : "=r"(l) : "f"(rb), "f"(ra));
  else asm("cvt.rz.f16x2.f32 %0, %1, %2;" : "=r"(l) : "f"(rb), "f"(ra));
  if constexpr (FLAGS) {  // only when the caller asked for range_flags
    const float aa = fabsf(a), ab = fabsf(b);
    // bit0: |x| >= 65520 (rounds to inf) or non-finite; bit1: 0 < |x| < 2^-3 (below 21-bit zone)
    flags |= (!(aa < 65520.f) || !(ab < 65520.f)) ? 1u : 0u;
    flags |= ((aa > 0.f && aa < 0.125f) || (ab > 0.f && ab < 0.125f)) ? 2u : 0u;
  }
  return SplitPair{h, l};
}

// Programmatic dependent launch (PDL) hooks.  Every split kernel lets its stream successor
// launch as soon as all of its CTAs are running (the tcgen05 GEMM that consumes the parts then
// sets up -- barriers, TMEM, tensor-map prefetch -- under the split's tail and waits with
// griddepcontrol.wait before its first operand load).  A split launched as the PDL follower
// of another, independent split (A's, then B's, in one egemm_gemm call) may run beside that
// split's tail; it waits for it at its END, so its own completion still implies the
// completion of everything before it in the stream (the GEMM's wait covers both splits).
// In a kernel that was not launched as a programmatic dependent, griddepcontrol.wait
// returns at once.
__device__ __forceinline__ void pdl_trigger() { asm volatile("griddepcontrol.launch_dependents;" ::: "memory"); }
__device__ __forceinline__ void pdl_wait_prev() { asm volatile("griddepcontrol.wait;" ::: "memory"); }

template <typename... KArgs, typename... Args>
static void launch_k(void (*k)(KArgs...), dim3 grid, cudaStream_t stream, bool pdl, Args... args) {
  cudaLaunchConfig_t c = {};
  c.gridDim = grid;
  c.blockDim = dim3(256, 1, 1);
  c.stream = stream;
  cudaLaunchAttribute a[1];
  a[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  a[0].val.programmaticStreamSerializationAllowed = 1;
  c.attrs = a;
  c.numAttrs = pdl ? 1 : 0;
  cudaLaunchKernelEx(&c, k, static_cast<KArgs>(args)...);
}

__device__ __forceinline__ void flush_flags(uint32_t flags, uint32_t* range_flags) {
  if (range_flags == nullptr) return;
  uint32_t any = __reduce_or_sync(0xffffffffu, flags);
  if (any && (threadIdx.x & 31) == 0) atomicOr(range_flags, any);
}

// Contiguous x, hi, lo: 8 elements per thread-iteration, scalar tail.
template <int MODE, bool FLAGS>
__global__ void __launch_bounds__(256) split_flat_kernel(const float* __restrict__ x, int64_t n,
                                                          uint16_t* __restrict__ hi,
                                                          uint16_t* __restrict__ lo,
                                                          uint32_t* range_flags) {
  pdl_trigger();
  uint32_t flags = 0;
  const int64_t nv = n >> 3;  // groups of 8: 2 x 16 B in, 16 B + 16 B out
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  for (int64_t g = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; g < nv; g += stride) {
    const float4* src = reinterpret_cast<const float4*>(x) + 2 * g;
    const float4 a = __ldcs(src), b = __ldcs(src + 1);
    const SplitPair p0 = split2<MODE, FLAGS>(a.x, a.y, flags), p1 = split2<MODE, FLAGS>(a.z, a.w, flags);
    const SplitPair p2 = split2<MODE, FLAGS>(b.x, b.y, flags), p3 = split2<MODE, FLAGS>(b.z, b.w, flags);
    __stcs(reinterpret_cast<uint4*>(hi) + g, make_uint4(p0.hi, p1.hi, p2.hi, p3.hi));
    __stcs(reinterpret_cast<uint4*>(lo) + g, make_uint4(p0.lo, p1.lo, p2.lo, p3.lo));
  }
  if (blockIdx.x == 0) {  // scalar tail (n % 8 elements)
    const int64_t t = (nv << 3) + threadIdx.x;
    if (t < n) {
      SplitPair p = split2<MODE>(x[t], 0.f, flags);
      hi[t] = (uint16_t)(p.hi & 0xffffu);
      lo[t] = (uint16_t)(p.lo & 0xffffu);
    }
  }
  flush_flags(flags, range_flags);
  pdl_wait_prev();
}

// Strided, same orientation: one thread per element.
template <int MODE>
__global__ void __launch_bounds__(256) split_strided_kernel(const float* __restrict__ x,
                                                             int64_t rows, int64_t cols,
                                                             int64_t ldx, uint16_t* __restrict__ hi,
                                                             uint16_t* __restrict__ lo,
                                                             int64_t ldo, uint32_t* range_flags) {
  pdl_trigger();
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
  pdl_wait_prev();
}

// Transposing: x is rows x cols (ldx); hi/lo are cols x rows (ldo).  64 x 64 tiles:
// coalesced loads along x's rows, split, transposed through shared memory (33-word pitch:
// conflict-light column writes), 4-B stores along the output rows.
constexpr int kTR = 64, kTC = 64;

template <int MODE>
__global__ void __launch_bounds__(256) split_transpose_kernel(const float* __restrict__ x,
                                                               int64_t rows, int64_t cols,
                                                               int64_t ldx,
                                                               uint16_t* __restrict__ hi,
                                                               uint16_t* __restrict__ lo,
                                                               int64_t ldo, uint32_t* range_flags,
                                                               int skip_full) {
  pdl_trigger();
  __shared__ uint32_t th[64][33];  // packed fp16 pairs of tile element [c][r]
  __shared__ uint32_t tl[64][33];
  uint32_t flags = 0;
  const int64_t r0 = (int64_t)blockIdx.y * kTR, c0 = (int64_t)blockIdx.x * kTC;
  if (skip_full && r0 + kTR <= rows && c0 + kTC <= cols) {  // done by the fast kernel
    pdl_wait_prev();
    return;
  }
  const int tx = threadIdx.x & 31, ty = threadIdx.x >> 5;  // 32 x 8
  for (int i = 0; i < 8; i++) {
    const int r = ty + 8 * i;
    const int64_t gr = r0 + r, gc = c0 + 2 * tx;
    float a = 0.f, b = 0.f;
    if (gr < rows) {
      if (gc < cols) a = x[gr * ldx + gc];
      if (gc + 1 < cols) b = x[gr * ldx + gc + 1];
    }
    const SplitPair p = split2<MODE>(a, b, flags);
    reinterpret_cast<uint16_t*>(&th[2 * tx][0])[r] = (uint16_t)(p.hi & 0xffffu);
    reinterpret_cast<uint16_t*>(&th[2 * tx + 1][0])[r] = (uint16_t)(p.hi >> 16);
    reinterpret_cast<uint16_t*>(&tl[2 * tx][0])[r] = (uint16_t)(p.lo & 0xffffu);
    reinterpret_cast<uint16_t*>(&tl[2 * tx + 1][0])[r] = (uint16_t)(p.lo >> 16);
  }
  __syncthreads();
  for (int i = 0; i < 8; i++) {  // output row = column c of x; 2 fp16 per thread
    const int c = ty + 8 * i;
    const int64_t oc = c0 + c, orow = r0 + 2 * tx;
    if (oc >= cols) continue;
    const uint32_t vh = th[c][tx], vl = tl[c][tx];
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
  flush_flags(flags, range_flags);  // padding elements are 0: they raise no flag
  pdl_wait_prev();
}

// Transposing, full 64 x 64 tiles with aligned rows (x: 16-B float4 loads; hi / lo: 16-B
// stores).  Each thread splits the PAIR (x[r][c], x[r+1][c]) into one packed fp16x2 word
// per output -- already the output's order along r -- so the smem transpose moves 32-bit
// words and the write-out is one 16-B store per 8 outputs.  Edge tiles (and unaligned
// operands) take split_transpose_kernel.
template <int MODE, bool FLAGS>
__global__ void __launch_bounds__(256) split_transpose_fast_kernel(
    const float* __restrict__ x, int64_t rows, int64_t cols, int64_t ldx, uint16_t* __restrict__ hi,
    uint16_t* __restrict__ lo, int64_t ldo, uint32_t* range_flags) {
  pdl_trigger();
  __shared__ uint32_t th[kTC][kTR / 2 + 1];  // [c][r/2]: packed (r, r+1) pairs, 33-word pitch
  __shared__ uint32_t tl[kTC][kTR / 2 + 1];
  uint32_t flags = 0;
  const int64_t r0 = (int64_t)blockIdx.y * kTR, c0 = (int64_t)blockIdx.x * kTC;
  const int t = threadIdx.x;
  {
    const int tx = t & 15, ty = t >> 4;  // 16 column quads x 16 row pairs (two passes)
#pragma unroll
    for (int i = 0; i < 2; i++) {
      const int rp = ty + 16 * i;  // row pair: rows 2 rp, 2 rp + 1
      const float* src = x + (r0 + 2 * rp) * ldx + c0 + 4 * tx;
      const float4 u = __ldcs(reinterpret_cast<const float4*>(src));
      const float4 v = __ldcs(reinterpret_cast<const float4*>(src + ldx));
      const SplitPair p0 = split2<MODE, FLAGS>(u.x, v.x, flags);
      const SplitPair p1 = split2<MODE, FLAGS>(u.y, v.y, flags);
      const SplitPair p2 = split2<MODE, FLAGS>(u.z, v.z, flags);
      const SplitPair p3 = split2<MODE, FLAGS>(u.w, v.w, flags);
      th[4 * tx][rp] = p0.hi; th[4 * tx + 1][rp] = p1.hi; th[4 * tx + 2][rp] = p2.hi; th[4 * tx + 3][rp] = p3.hi;
      tl[4 * tx][rp] = p0.lo; tl[4 * tx + 1][rp] = p1.lo; tl[4 * tx + 2][rp] = p2.lo; tl[4 * tx + 3][rp] = p3.lo;
    }
  }
  __syncthreads();
#pragma unroll
  for (int i = 0; i < 2; i++) {  // 64 output rows x 8 chunks of 8 fp16 = 512 chunks
    const int q = t + 256 * i;
    const int c = q >> 3, k = q & 7;
    const uint4 vh = make_uint4(th[c][4 * k], th[c][4 * k + 1], th[c][4 * k + 2], th[c][4 * k + 3]);
    const uint4 vl = make_uint4(tl[c][4 * k], tl[c][4 * k + 1], tl[c][4 * k + 2], tl[c][4 * k + 3]);
    const int64_t o = (c0 + c) * ldo + r0 + 8 * k;
    __stcs(reinterpret_cast<uint4*>(hi + o), vh);
    __stcs(reinterpret_cast<uint4*>(lo + o), vl);
  }
  if constexpr (FLAGS) flush_flags(flags, range_flags);
  pdl_wait_prev();
}

template <int MODE>
static void launch_mode(const float* x, int64_t rows, int64_t cols, int64_t ldx, uint16_t* hi,
                        uint16_t* lo, int64_t ldo, int transpose, uint32_t* range_flags,
                        cudaStream_t stream, bool pdl) {
  const int nsm = num_sms();
  const bool fl = range_flags != nullptr;
  if (!transpose) {
    const bool flat = (ldx == cols && ldo == cols && ((uintptr_t)x % 16 == 0) &&
                       ((uintptr_t)hi % 16 == 0) && ((uintptr_t)lo % 16 == 0));
    const int64_t n = rows * cols;
    if (flat) {
      int64_t blocks = ((n >> 3) + 255) / 256;
      const int64_t cap = (int64_t)nsm * 8;  // 8 x 256 threads resident per SM
      if (blocks > cap) blocks = cap;
      if (blocks < 1) blocks = 1;
      if (fl) launch_k(split_flat_kernel<MODE, true>, dim3((unsigned)blocks), stream, pdl, x, n, hi, lo, range_flags);
      else launch_k(split_flat_kernel<MODE, false>, dim3((unsigned)blocks), stream, pdl, x, n, hi, lo, nullptr);
    } else {
      int64_t blocks = (n + 255) / 256;
      const int64_t cap = (int64_t)nsm * 8;
      if (blocks > cap) blocks = cap;
      launch_k(split_strided_kernel<MODE>, dim3((unsigned)blocks), stream, pdl, x, rows, cols, ldx, hi,
               lo, ldo, range_flags);
    }
  } else {
    dim3 grid((unsigned)((cols + kTC - 1) / kTC), (unsigned)((rows + kTR - 1) / kTR));
    const bool fast = (ldx % 4 == 0) && ((uintptr_t)x % 16 == 0) && (ldo % 8 == 0) &&
                      ((uintptr_t)hi % 16 == 0) && ((uintptr_t)lo % 16 == 0);
    const dim3 full((unsigned)(cols / kTC), (unsigned)(rows / kTR));
    bool launched = false;
    if (fast && full.x > 0 && full.y > 0) {
      if (fl)
        launch_k(split_transpose_fast_kernel<MODE, true>, full, stream, pdl, x, rows, cols, ldx, hi, lo,
                 ldo, range_flags);
      else
        launch_k(split_transpose_fast_kernel<MODE, false>, full, stream, pdl, x, rows, cols, ldx, hi, lo,
                 ldo, nullptr);
      launched = true;
    }
    const bool edges = !fast || (cols % kTC) != 0 || (rows % kTR) != 0 || full.x == 0 || full.y == 0;
    // the edge tiles are independent of the full ones: a PDL follower of the fast kernel
    if (edges)
      launch_k(split_transpose_kernel<MODE>, grid, stream, pdl || launched, x, rows, cols, ldx, hi,
               lo, ldo, range_flags, fast ? 1 : 0);
  }
}

int launch_split(const float* x, int64_t rows, int64_t cols, int64_t ldx, uint16_t* hi,
                 uint16_t* lo, int64_t ldo, int transpose, uint32_t* range_flags,
                 cudaStream_t stream, int mode, bool pdl) {
  if (rows == 0 || cols == 0) return 0;
  if (mode == 1) launch_mode<1>(x, rows, cols, ldx, hi, lo, ldo, transpose, range_flags, stream, pdl);
  else if (mode == 2) launch_mode<2>(x, rows, cols, ldx, hi, lo, ldo, transpose, range_flags, stream, pdl);
  else launch_mode<0>(x, rows, cols, ldx, hi, lo, ldo, transpose, range_flags, stream, pdl);
  return cudaGetLastError() == cudaSuccess ? 0 : -1;
}

}  // namespace egemm
