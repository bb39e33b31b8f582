// Instantiations of msv_fast_kernel<32, Q> and msv_multi_kernel<32, Q> for Q = 1..40 (one file per G so nvcc runs in parallel).
#include "msv_multi.cuh"

namespace hmg {
namespace {
template <int Q>
const void* pick(int q) {
  if constexpr (Q > 40) {
    return nullptr;
  } else {
    if (q == Q) return msv_fast_entry<32, Q>();
    return pick<Q + 1>(q);
  }
}
template <int Q>
const void* pick_multi(int q) {
  if constexpr (Q > 40) {
    return nullptr;
  } else {
    if (q == Q) return msv_multi_entry<32, Q>();
    return pick_multi<Q + 1>(q);
  }
}
}  // namespace
const void* msv_fast_ptr_g32(int q) { return pick<1>(q); }
const void* msv_multi_ptr_g32(int q) { return pick_multi<1>(q); }
}  // namespace hmg
