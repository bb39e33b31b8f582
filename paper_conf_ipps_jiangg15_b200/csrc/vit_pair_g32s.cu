// Instantiations of vit_pair_kernel<32, Q, SCAN = true> for Q = 1..16 (max-plus scan Lazy-F).
#include "vit_pair.cuh"

namespace hmg {
namespace {
template <int Q>
const void* pick(int q) {
  if constexpr (Q > 16) {
    return nullptr;
  } else {
    if (q == Q) return reinterpret_cast<const void*>(&vit_pair_kernel<32, Q, true>);
    return pick<Q + 1>(q);
  }
}
}  // namespace
const void* vit_pair_ptr_g32s(int q) { return pick<1>(q); }
}  // namespace hmg
