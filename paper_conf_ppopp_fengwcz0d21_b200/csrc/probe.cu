// probe.cu -- the paper's tensor-core precision profiling (Sec. 3.1, PAPER.md P:596-649:
// feed designed inputs through the real MMA, compare bitwise against CPU "probing
// primitives") generalised to every floating tcgen05 kind the emulation could be built on
// (SURVEY §8(f) NEXT-3): kind::f16 with fp16 or bf16 operands and kind::tf32, fp32 D.
//
// One CTA, cta_group::1, M = 128: D[128 x N] = C + sum_k A[:, k] B[:, k]^T as ONE chain of
// tcgen05.mma instructions over K (16 fp16/bf16 or 8 tf32 elements each), C loaded into the
// TMEM accumulator first with tcgen05.st.  Operands are copied into the same 128-B-swizzled
// K-major smem layout the GEMM's TMA writes, by plain loads/stores (this is a probe, not a
// fast path).  Diagnostics / profiling only; the GEMM does not call it.
#include <cuda_runtime.h>
#include <cstdint>
#include "egemm_internal.h"
#include "ptx.cuh"

namespace egemm {

constexpr int kProbeM = 128;

template <int KIND>  // 0: f16 x f16, 1: bf16 x bf16 (both kind::f16), 2: tf32 x tf32 (kind::tf32)
__device__ __forceinline__ void probe_mma(uint32_t d, uint64_t a, uint64_t b, uint32_t idesc,
                                          uint32_t acc) {
  if constexpr (KIND == 2) {
    asm volatile(
        "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
        "tcgen05.mma.cta_group::1.kind::tf32 [%0], %1, %2, %3, p;\n\t}" ::"r"(d),
        "l"(a), "l"(b), "r"(idesc), "r"(acc));
  } else {
    asm volatile(
        "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
        "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(d),
        "l"(a), "l"(b), "r"(idesc), "r"(acc));
  }
}

__device__ __forceinline__ void tmem_st32(uint32_t taddr, const float* v) {
  const uint32_t* r = reinterpret_cast<const uint32_t*>(v);
  asm volatile(
      "tcgen05.st.sync.aligned.32x32b.x32.b32 [%0], {%1, %2, %3, %4, %5, %6, %7, %8, %9, %10, "
      "%11, %12, %13, %14, %15, %16, %17, %18, %19, %20, %21, %22, %23, %24, %25, %26, %27, "
      "%28, %29, %30, %31, %32};" ::"r"(taddr),
      "r"(r[0]), "r"(r[1]), "r"(r[2]), "r"(r[3]), "r"(r[4]), "r"(r[5]), "r"(r[6]), "r"(r[7]),
      "r"(r[8]), "r"(r[9]), "r"(r[10]), "r"(r[11]), "r"(r[12]), "r"(r[13]), "r"(r[14]),
      "r"(r[15]), "r"(r[16]), "r"(r[17]), "r"(r[18]), "r"(r[19]), "r"(r[20]), "r"(r[21]),
      "r"(r[22]), "r"(r[23]), "r"(r[24]), "r"(r[25]), "r"(r[26]), "r"(r[27]), "r"(r[28]),
      "r"(r[29]), "r"(r[30]), "r"(r[31])
      : "memory");
  asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
}

// Copy a rows x K row-major operand (element bytes EB) into the swizzled K-major layout:
// k-blocks of 128 B per row, 8-row atoms, 16-B chunk c of row r stored at chunk c ^ (r & 7).
template <int EB>
__device__ void probe_stage(const uint8_t* src, int rows, int K, int kblocks, uint8_t* dst) {
  const int chunks = rows * kblocks * 8;  // 16-B chunks
  for (int i = threadIdx.x; i < chunks; i += blockDim.x) {
    const int c = i & 7, r = (i >> 3) % rows, kb = (i >> 3) / rows;
    uint8_t buf[16];
#pragma unroll
    for (int e = 0; e < 16 / EB; e++) {
      const int k = kb * (128 / EB) + c * (16 / EB) + e;
#pragma unroll
      for (int b = 0; b < EB; b++)
        buf[e * EB + b] = (k < K) ? src[((int64_t)r * K + k) * EB + b] : (uint8_t)0;
    }
    uint8_t* o = dst + (size_t)kb * rows * 128 + r * 128 + ((c ^ (r & 7)) << 4);
#pragma unroll
    for (int b = 0; b < 16; b++) o[b] = buf[b];
  }
}

template <int KIND>
__global__ void __launch_bounds__(128) tc_probe_kernel(const uint8_t* A, const uint8_t* B,
                                                       const float* C, float* D, int N, int K) {
  constexpr int EB = (KIND == 2) ? 4 : 2;
  constexpr int KSTEP = 32 / EB;     // elements per MMA
  constexpr int STEPS_KB = 128 / 32;  // MMAs per 128-B k-block
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) &
                                             ~uintptr_t(1023));
  const int kblocks = (K * EB + 127) / 128;
  uint8_t* sa = smem;
  uint8_t* sb = sa + (size_t)kblocks * kProbeM * 128;
  uint64_t* bar = reinterpret_cast<uint64_t*>(sb + (size_t)kblocks * N * 128);
  uint32_t* slot = reinterpret_cast<uint32_t*>(bar + 1);
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;

  probe_stage<EB>(A, kProbeM, K, kblocks, sa);
  probe_stage<EB>(B, N, K, kblocks, sb);
  ptx::fence_proxy_async_smem();
  if (threadIdx.x == 0) {
    ptx::mbar_init(bar, 1);
    ptx::fence_mbar_init();
  }
  if (warp == 0) ptx::tmem_alloc<1>(slot, 256);
  ptx::tc_fence_before();
  __syncthreads();
  ptx::tc_fence_after();
  const uint32_t tmem = *slot;
  const int row = warp * 32 + lane;
  const uint32_t lane_off = (uint32_t)(warp * 32) << 16;
  if (C) {  // the addend goes into the accumulator before the first MMA
    for (int c0 = 0; c0 < N; c0 += 32) {
      float v[32];
#pragma unroll
      for (int j = 0; j < 32; j++) v[j] = (c0 + j < N) ? C[(int64_t)row * N + c0 + j] : 0.f;
      tmem_st32(tmem + lane_off + c0, v);
    }
  }
  ptx::tc_fence_before();
  __syncthreads();
  ptx::tc_fence_after();
  if (threadIdx.x == 0) {
    const uint32_t idesc = (1u << 4) | ((uint32_t)(KIND == 1 ? 1 : KIND == 2 ? 2 : 0) << 7) |
                           ((uint32_t)(KIND == 1 ? 1 : KIND == 2 ? 2 : 0) << 10) |
                           ((uint32_t)(N >> 3) << 17) | ((uint32_t)(kProbeM >> 4) << 24);
    const int steps = (K + KSTEP - 1) / KSTEP;
    for (int s = 0; s < steps; s++) {
      const int kb = s / STEPS_KB, w = s % STEPS_KB;
      const uint64_t ad = ptx::sdesc_kmajor_sw128(ptx::smem_u32(sa + (size_t)kb * kProbeM * 128)) +
                          (uint64_t)(w * 2);
      const uint64_t bd = ptx::sdesc_kmajor_sw128(ptx::smem_u32(sb + (size_t)kb * N * 128)) +
                          (uint64_t)(w * 2);
      probe_mma<KIND>(tmem, ad, bd, idesc, (C != nullptr || s > 0) ? 1u : 0u);
    }
    ptx::mma_commit<1>(bar);
  }
  ptx::mbar_wait(bar, 0);
  ptx::tc_fence_after();
  for (int c0 = 0; c0 < N; c0 += 32) {
    float v[32];
    ptx::tmem_ld32(tmem + lane_off + c0, v);
    ptx::tmem_wait_ld();
#pragma unroll
    for (int j = 0; j < 32; j++)
      if (c0 + j < N) D[(int64_t)row * N + c0 + j] = v[j];
  }
  ptx::tc_fence_before();
  __syncthreads();
  if (warp == 0) {
    ptx::tc_fence_after();
    ptx::tmem_dealloc<1>(tmem, 256);
  }
}

size_t tc_probe_smem(int kind, int N, int K) {
  const int eb = (kind == 2) ? 4 : 2;
  const size_t kblocks = ((size_t)K * eb + 127) / 128;
  return kblocks * (kProbeM + N) * 128 + 64 + 1024;
}

int launch_tc_probe(int kind, int N, int K, const void* A, const void* B, const float* C,
                    float* D, cudaStream_t stream) {
  const size_t smem = tc_probe_smem(kind, N, K);
  const uint8_t* a = static_cast<const uint8_t*>(A);
  const uint8_t* b = static_cast<const uint8_t*>(B);
  cudaError_t e;
  if (kind == 0) {
    cudaFuncSetAttribute(tc_probe_kernel<0>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    tc_probe_kernel<0><<<1, 128, smem, stream>>>(a, b, C, D, N, K);
  } else if (kind == 1) {
    cudaFuncSetAttribute(tc_probe_kernel<1>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    tc_probe_kernel<1><<<1, 128, smem, stream>>>(a, b, C, D, N, K);
  } else {
    cudaFuncSetAttribute(tc_probe_kernel<2>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    tc_probe_kernel<2><<<1, 128, smem, stream>>>(a, b, C, D, N, K);
  }
  e = cudaGetLastError();
  return e == cudaSuccess ? 0 : -1;
}

}  // namespace egemm
