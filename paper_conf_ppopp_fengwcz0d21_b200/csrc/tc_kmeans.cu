// tc_kmeans.cu -- the kMeans variants of the tensor-core kernel (fused argmin epilogue, the
// kMeans case study): CTA pair 256 x 256 or single CTA 128 x 128, 16 or 8
// epilogue warps (the argmin epilogue is issue-bound next to a 64-deep k-loop).
#include "tc_kernel.cuh"

namespace egemm {

int dispatch_kmeans(const CUtensorMap* m, const KParams& kp, const TcConfig& c, cudaStream_t s) {
  const int mc = c.max_clusters;
  const bool e8 = c.nepi == 8;
  if (c.cg == 2 && c.bn == 256) {
    if (e8) return launch_variant<2, 256, false, EPI_KMEANS, 3, false, false, false, false, 8>(m, kp, mc, s);
    return launch_variant<2, 256, false, EPI_KMEANS, 3, false, false, false, false, 16>(m, kp, mc, s);
  }
  if (c.cg == 1 && c.bn == 128) {
    if (e8) return launch_variant<1, 128, false, EPI_KMEANS, 3, false, false, false, false, 8>(m, kp, mc, s);
    return launch_variant<1, 128, false, EPI_KMEANS, 3, false, false, false, false, 16>(m, kp, mc, s);
  }
  set_last_error("kMeans: unsupported tile config cg=%d bn=%d", c.cg, c.bn);
  return 2;
}

}  // namespace egemm
