// Instantiations of fwd_kernel<1, Q, S> for Q = 2, 4, 8, 12, 13, 14, 16 and S = 2, 4, 8, 12, and of the
// sub-warp lane-group kernels fwd_kernel<1, Q, S, 8> (Q = 2, 4).
#include "forward.cuh"

namespace hmg {
namespace {
template <int Q>
const void* pick_s(int s) {
  if (Q >= 12 && 32 * 1 * s > 256) return nullptr;   // 12-16 nodes/thread need ~200-250 registers
  if (s == 2) return reinterpret_cast<const void*>(&fwd_kernel<1, Q, 2>);
  if (s == 4) return reinterpret_cast<const void*>(&fwd_kernel<1, Q, 4>);
  if (s == 8) return reinterpret_cast<const void*>(&fwd_kernel<1, Q, 8>);
  if (s == 12) return reinterpret_cast<const void*>(&fwd_kernel<1, Q, 12>);
  return nullptr;
}
// sub-warp lane groups (GL = 8 lanes per sequence), S sequences per block
template <int Q, int GL>
const void* pick_g(int s) {
  if (GL * s > 256) return nullptr;              // > 256 threads would cap registers at 128
  if (s == 4) return reinterpret_cast<const void*>(&fwd_kernel<1, Q, 4, GL>);
  if (s == 8) return reinterpret_cast<const void*>(&fwd_kernel<1, Q, 8, GL>);
  if (s == 16) return reinterpret_cast<const void*>(&fwd_kernel<1, Q, 16, GL>);
  if (s == 32) return reinterpret_cast<const void*>(&fwd_kernel<1, Q, 32, GL>);
  return nullptr;
}
}  // namespace
const void* fwd_ptr_sub(int gl, int q, int s) {
  if (gl == 8) {
    switch (q) {
      case 2: return pick_g<2, 8>(s);
      case 4: return pick_g<4, 8>(s);
    }
  }
  return nullptr;
}
const void* fwd_ptr_w1(int q, int s) {
  switch (q) {
    case 2: return pick_s<2>(s);
    case 4: return pick_s<4>(s);
    case 8: return pick_s<8>(s);
    case 12: return pick_s<12>(s);
    case 13: return pick_s<13>(s);
    case 14: return pick_s<14>(s);
    case 16: return pick_s<16>(s);
  }
  return nullptr;
}
}  // namespace hmg
