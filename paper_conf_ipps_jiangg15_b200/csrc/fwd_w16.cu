// Instantiations of fwd_kernel<16, Q, S> for Q = 2, 4, 8 and S = 1.
#include "forward.cuh"

namespace hmg {
namespace {
template <int Q>
const void* pick_s(int s) {
  if (s == 1) return reinterpret_cast<const void*>(&fwd_kernel<16, Q, 1>);
  return nullptr;
}
}  // namespace
const void* fwd_ptr_w16(int q, int s) {
  switch (q) {
    case 2: return pick_s<2>(s);
    case 4: return pick_s<4>(s);
    case 8: return pick_s<8>(s);
  }
  return nullptr;
}
}  // namespace hmg
