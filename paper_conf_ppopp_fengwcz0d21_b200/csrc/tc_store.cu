// tc_store.cu -- the STORE (D = A B + C) variants of the tensor-core kernel on pre-split
// operands: tile (cta_group, BN), accumulator mode (SEP) and smem ring depth, the axes of
// the measured tuning table.
#include "tc_kernel.cuh"

namespace egemm {

int dispatch_store(const CUtensorMap* m, const KParams& kp, const TcConfig& c, cudaStream_t s) {
  const int mc = c.max_clusters;
  const int st = c.stages;
  if (c.cg == 2 && c.bn == 256 && !c.sep) {  // 64 KiB stages
    if (st == 2) return launch_variant<2, 256, false, EPI_STORE, 2>(m, kp, mc, s);
    if (st == 0 || st == 3) return launch_variant<2, 256, false, EPI_STORE, 3>(m, kp, mc, s);
  } else if (c.cg == 2 && c.bn == 224 && !c.sep) {  // 60 KiB stages: ceil(N / 224) n-tiles
    if (st == 2) return launch_variant<2, 224, false, EPI_STORE, 2>(m, kp, mc, s);
    if (st == 0 || st == 3) return launch_variant<2, 224, false, EPI_STORE, 3>(m, kp, mc, s);
  } else if (c.cg == 2 && c.bn == 128 && !c.sep) {  // 48 KiB stages, one accumulator in ping-pong
    if (st == 3) return launch_variant<2, 128, false, EPI_STORE, 3>(m, kp, mc, s);
    if (st == 0 || st == 4) return launch_variant<2, 128, false, EPI_STORE, 4>(m, kp, mc, s);
  } else if (c.cg == 2 && c.bn == 128 && c.sep) {
    if (st == 4) return launch_variant<2, 128, true, EPI_STORE, 4>(m, kp, mc, s);
    if (st == 0 || st == 3) return launch_variant<2, 128, true, EPI_STORE, 3>(m, kp, mc, s);
  } else if (c.cg == 1 && c.bn == 128 && !c.sep) {  // 64 KiB stages (128 rows of A and B)
    if (st == 2) return launch_variant<1, 128, false, EPI_STORE, 2>(m, kp, mc, s);
    if (st == 0 || st == 3) return launch_variant<1, 128, false, EPI_STORE, 3>(m, kp, mc, s);
  } else if (c.cg == 1 && c.bn == 128 && c.sep) {
    if (st == 2) return launch_variant<1, 128, true, EPI_STORE, 2>(m, kp, mc, s);
    if (st == 0 || st == 3) return launch_variant<1, 128, true, EPI_STORE, 3>(m, kp, mc, s);
  }
  set_last_error("unsupported tile config cg=%d bn=%d sep=%d stages=%d", c.cg, c.bn, c.sep, st);
  return 2;
}

}  // namespace egemm
