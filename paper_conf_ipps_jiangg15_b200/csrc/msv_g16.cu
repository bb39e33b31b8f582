// Instantiations of msv_fast_kernel<16, Q> for Q = 1..32 (one file per G so nvcc runs in parallel).
#include "msv.cuh"

namespace hmg {
namespace {
template <int Q>
const void* pick(int q) {
  if constexpr (Q > 32) {
    return nullptr;
  } else {
    if (q == Q) return reinterpret_cast<const void*>(&msv_fast_kernel<16, Q>);
    return pick<Q + 1>(q);
  }
}
}  // namespace
const void* msv_fast_ptr_g16(int q) { return pick<1>(q); }
}  // namespace hmg
