// tc_knn.cu -- the kNN variants of the tensor-core kernel (fused distance + top-k epilogue,
// the kNN case study): list length KN in {16, 32, 64} (k <= KN), query tile
// resident in smem (d <= 128) or streamed, CTA pair 256 x 256 or single CTA 128 x 128.
#include "tc_kernel.cuh"

namespace egemm {

template <int KN>
static int knn_kn(const CUtensorMap* m, const KParams& kp, const TcConfig& c, cudaStream_t s) {
  const int mc = c.max_clusters;
  if (c.cg == 2 && c.bn == 256) {
    // the unit's (query) A tile stays resident across its reference tiles when d <= 128,
    // halving L2->smem traffic (measured +5 % q/s)
    if (kp.num_kb <= 2 && c.ares != 0 && !(kDiag && kp.debug_no_tma))
      return launch_variant<2, 256, false, EPI_KNN, 3, false, true, false, false, 8, KN>(m, kp, mc, s);
    return launch_variant<2, 256, false, EPI_KNN, 3, false, false, false, false, 8, KN>(m, kp, mc, s);
  }
  if constexpr (KN == 16) {
    if (c.cg == 1 && c.bn == 128)
      return launch_variant<1, 128, false, EPI_KNN, 3, false, false, false, false, 8, 16>(m, kp, mc, s);
  }
  set_last_error("kNN: unsupported tile config cg=%d bn=%d for k=%d", c.cg, c.bn, kp.knn_k);
  return 2;
}

int dispatch_knn(const CUtensorMap* m, const KParams& kp, const TcConfig& c, cudaStream_t s) {
  if (kp.knn_k <= 16) return knn_kn<16>(m, kp, c, s);
  if (kp.knn_k <= 32) return knn_kn<32>(m, kp, c, s);
  return knn_kn<64>(m, kp, c, s);
}

}  // namespace egemm
