// tc_kmeans.cu -- the kMeans variants of the tensor-core kernel (fused argmin epilogue, the
// kMeans case study): CTA pair 256 x 256 (point tile resident or streamed) or
// single CTA 128 x 128, 16 or 8 epilogue warps (the argmin epilogue is issue-bound next to a
// 64-deep k-loop).
#include "tc_kernel.cuh"

namespace egemm {

int dispatch_kmeans(const CUtensorMap* m, const KParams& kp, const TcConfig& c, cudaStream_t s) {
  const int mc = c.max_clusters;
  const bool e8 = c.nepi == 8;
  if (c.cg == 2 && c.bn == 256) {
    // AR (opt-in: a_resident = 1): a unit's point tile (d <= 128) stays resident across the
    // centroid tiles, so the ring carries only the centroids (L2 -> smem bytes per unit:
    // 4 x (A + B) -> A + 4 x B).  Measured the same cycles as streaming (the argmin epilogue,
    // not operand traffic, sets the pace: profiles/r02_kmeans_ar_ab.json), so not the default.
    if (kp.num_kb <= 2 && c.ares > 0 && !(kDiag && kp.debug_no_tma)) {
      if (e8) return launch_variant<2, 256, false, EPI_KMEANS, 3, false, true, false, false, 8>(m, kp, mc, s);
      return launch_variant<2, 256, false, EPI_KMEANS, 3, false, true, false, false, 16>(m, kp, mc, s);
    }
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
