// Instantiations of fwd_kernel<1, Q, S> for Q = 2, 4, 8 and S = 2, 4, 8, 12.
#include "forward.cuh"

namespace hmg {
namespace {
template <int Q>
const void* pick_s(int s) {
  if (s == 2) return reinterpret_cast<const void*>(&fwd_kernel<1, Q, 2>);
  if (s == 4) return reinterpret_cast<const void*>(&fwd_kernel<1, Q, 4>);
  if (s == 8) return reinterpret_cast<const void*>(&fwd_kernel<1, Q, 8>);
  if (s == 12) return reinterpret_cast<const void*>(&fwd_kernel<1, Q, 12>);
  return nullptr;
}
}  // namespace
const void* fwd_ptr_w1(int q, int s) {
  switch (q) {
    case 2: return pick_s<2>(s);
    case 4: return pick_s<4>(s);
    case 8: return pick_s<8>(s);
  }
  return nullptr;
}
}  // namespace hmg
