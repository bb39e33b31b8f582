// Instantiations of fwd_kernel<4, Q, S> for Q = 2, 4, 8, 16 and S = 1, 2, 3.
#include "forward.cuh"

namespace hmg {
namespace {
template <int Q>
const void* pick_s(int s) {
  if (Q == 16 && 32 * 4 * s > 256) return nullptr;   // 16 nodes/thread need ~250 registers
  if (s == 1) return reinterpret_cast<const void*>(&fwd_kernel<4, Q, 1>);
  if (s == 2) return reinterpret_cast<const void*>(&fwd_kernel<4, Q, 2>);
  if (s == 3) return reinterpret_cast<const void*>(&fwd_kernel<4, Q, 3>);
  return nullptr;
}
}  // namespace
const void* fwd_ptr_w4(int q, int s) {
  switch (q) {
    case 2: return pick_s<2>(s);
    case 4: return pick_s<4>(s);
    case 8: return pick_s<8>(s);
    case 16: return pick_s<16>(s);
  }
  return nullptr;
}
}  // namespace hmg
