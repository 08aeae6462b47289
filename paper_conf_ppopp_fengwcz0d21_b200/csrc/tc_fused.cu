// tc_fused.cu -- STORE variants with a round-split inside the GEMM (SURVEY 8a-2 fused mode):
// fp32 A converted by a converter warpgroup (LDG, or TMA-staged and converted in place), or
// fp32 B (TMA-staged, transposed to K-major on the way).
#include "tc_kernel.cuh"

namespace egemm {

int dispatch_fused(const CUtensorMap* m, const KParams& kp, const TcConfig& c, cudaStream_t s) {
  const int mc = c.max_clusters;
  if (kp.fb) {  // fused B split: TMA-staged fp32 B (2 MMA stages + 3 fp32 staging slots)
    if (c.cg == 2 && c.bn == 256 && !c.sep)
      return launch_variant<2, 256, false, EPI_STORE, 2, false, false, false, true>(m, kp, mc, s);
    if (c.cg == 2 && c.bn == 224 && !c.sep)
      return launch_variant<2, 224, false, EPI_STORE, 2, false, false, false, true>(m, kp, mc, s);
    set_last_error("fused B split: unsupported tile config cg=%d bn=%d sep=%d", c.cg, c.bn, c.sep);
    return 2;
  }
  // fused A: aligned fp32 A is TMA-staged into the stage's A region and split in place;
  // otherwise the LDG converters
  if (c.cg == 2 && c.bn == 256 && !c.sep && kp.a_staged) {
    if (c.stages == 2) return launch_variant<2, 256, false, EPI_STORE, 2, true, false, true>(m, kp, mc, s);
    return launch_variant<2, 256, false, EPI_STORE, 3, true, false, true>(m, kp, mc, s);
  }
  if (c.cg == 2 && c.bn == 256 && !c.sep)
    return launch_variant<2, 256, false, EPI_STORE, 3, true>(m, kp, mc, s);
  if (c.cg == 2 && c.bn == 128 && c.sep)
    return launch_variant<2, 128, true, EPI_STORE, 3, true>(m, kp, mc, s);
  if (c.cg == 2 && c.bn == 128 && !c.sep)
    return launch_variant<2, 128, false, EPI_STORE, 3, true>(m, kp, mc, s);
  if (c.cg == 1 && c.bn == 128 && c.sep)
    return launch_variant<1, 128, true, EPI_STORE, 3, true>(m, kp, mc, s);
  if (c.cg == 1 && c.bn == 128 && !c.sep)  // (the peeled tail of a (2, 256, 0) fused-A call)
    return launch_variant<1, 128, false, EPI_STORE, 3, true>(m, kp, mc, s);
  set_last_error("fused A split: unsupported tile config cg=%d bn=%d sep=%d", c.cg, c.bn, c.sep);
  return 2;
}

}  // namespace egemm
