// Diagnostics only (tools/diag_gemm.py): one warp that spins for `ns` nanoseconds of
// %globaltimer and records the SM cycles (clock64) it saw -- launched on a side stream it
// co-resides with a running GEMM (32 threads, no shared memory) and measures the SM clock
// the GEMM actually ran at.
#include <cuda_runtime.h>
#include <cstdint>

__device__ unsigned long long g_spin[2];

__global__ void clockspin_kernel(unsigned long long ns) {
  unsigned long long t0, t, c0 = clock64();
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t0));
  do {
    __nanosleep(1000);
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  } while (t - t0 < ns);
  if (threadIdx.x == 0) {
    g_spin[0] = clock64() - c0;
    g_spin[1] = t - t0;
  }
}

extern "C" int clockspin_launch(double ms, void* stream) {
  clockspin_kernel<<<1, 32, 0, (cudaStream_t)stream>>>((unsigned long long)(ms * 1e6));
  return (int)cudaGetLastError();
}

extern "C" int clockspin_read(double* mhz) {
  unsigned long long h[2];
  int e = (int)cudaMemcpyFromSymbol(h, g_spin, sizeof(h));
  *mhz = h[1] ? (double)h[0] * 1e3 / (double)h[1] : 0.0;
  return e;
}
