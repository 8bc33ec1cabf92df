// Thread-per-query scan with a runtime padded dimension (dp > 32), used for
// large k where the warp-per-query lane-distributed top-k (k <= 32) cannot be.
#include "k_scan_tpq.cuh"

namespace sknn {
template void launch_tpq_dp<0>(Ctx& cx, const ScanArgs& a);
}  // namespace sknn
