// Instantiations of fwd_kernel<1, Q, S> for Q = 2, 4, 8, 16 and S = 2, 4, 8, 12.
#include "forward.cuh"

namespace hmg {
namespace {
template <int Q>
const void* pick_s(int s) {
  if (Q == 16 && 32 * 1 * s > 256) return nullptr;   // 16 nodes/thread need ~250 registers
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
    case 16: return pick_s<16>(s);
  }
  return nullptr;
}
}  // namespace hmg
