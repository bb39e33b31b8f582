// Instantiations of msv_fast_kernel<4, Q> and msv_multi_kernel<4, Q> for Q = 1..32 (one file per G so nvcc runs in parallel).
#include "msv_multi.cuh"

namespace hmg {
namespace {
template <int Q>
const void* pick(int q) {
  if constexpr (Q > 32) {
    return nullptr;
  } else {
    if (q == Q) return msv_fast_entry<4, Q>();
    return pick<Q + 1>(q);
  }
}
template <int Q>
const void* pick_multi(int q) {
  if constexpr (Q > 32) {
    return nullptr;
  } else {
    if (q == Q) return msv_multi_entry<4, Q>();
    return pick_multi<Q + 1>(q);
  }
}
}  // namespace
const void* msv_fast_ptr_g4(int q) { return pick<1>(q); }
const void* msv_multi_ptr_g4(int q) { return pick_multi<1>(q); }
}  // namespace hmg
