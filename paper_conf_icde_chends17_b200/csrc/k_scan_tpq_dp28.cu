// Explicit instantiation of the thread-per-query scan for padded dimension 28
// (split across files so nvcc compiles the 8 x 8 template grid in parallel).
#include "k_scan_tpq.cuh"

namespace sknn {
template void launch_tpq_dp<28>(Ctx& cx, const ScanArgs& a);
}  // namespace sknn
