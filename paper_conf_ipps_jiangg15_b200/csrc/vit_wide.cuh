// vit_wide.cuh -- Viterbi filter (Alg 2, + Lazy-F, P:519-533 / Fig 7) for long models
// (up to 2048 nodes) with ONE warp per sequence and two cells per register: the lane of
// vit_pair.cuh (VitPairLane: s16x2 offset arithmetic, Farrar striping over 64 virtual lanes,
// vote-terminated D->D carry passes) with Q up to 32 registers per lane.
//
// 32 registers per lane of M, I, D and the B->M terms leave no room for the seven transition
// vectors (7 x 32 registers), so the five the M / I updates use (tMM, tIM, tDM, tMI, tII) are read
// per row from shared memory (one copy per block, the load_row chunk layout, LDS.128 per four
// registers) and only the D chain's tMD and tDD stay in registers.  The row is processed in
// chunks of four registers, highest first (M(i,k) needs the unchanged M(i-1,k-1)).  No barrier
// at all: the sequence's row lives in one warp, so an SM holds eight independent sequences (two
// 128-thread blocks of four warps, ~104 KB of shared memory each) where the two-warp kernel
// (vit_cpair2.cuh) holds four.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include "hmg_internal.h"
#include "msv.cuh"        // ResStream
#include "vit_pair.cuh"   // kRedo

namespace hmg {

// tMD is streamed from shared memory too above 24 registers (the 32-register lane spilled)
template <int Q> constexpr bool wide_tmd_smem() { return Q > 24; }

// shared-memory LDS.128 of four transition registers.  Up to 20 registers per lane the loads are
// plain (the compiler schedules them early: 1948 -> 2314 GCUPS at M = 1100); above, they are
// volatile, i.e. kept in program order, or the hoisted loads spill the 255-register lane
// (933 GCUPS at M = 2048; profiles/wide_r02w.jsonl)
template <bool ORDERED>
__device__ __forceinline__ uint4 lds4(uint32_t addr) {
  uint4 v;
  if constexpr (ORDERED)
    asm volatile("ld.shared.v4.u32 {%0, %1, %2, %3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "r"(addr));
  else
    asm("ld.shared.v4.u32 {%0, %1, %2, %3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "r"(addr));
  return v;
}

template <int Q, bool TM>
struct VitWideSmem {
  static_assert(Q % 4 == 0, "chunks of four registers");
  static constexpr int ROWW = Q * 32;            // s16x2 words per residue row / per vector
  static constexpr int SROWS = 21;               // 20 canonical residues + X (code 26)
  // tMM, tIM, tDM, tMI, tII (+ tMD) in shared memory; none with the tensor-memory copy
  static constexpr int TROWS = TM ? 0 : wide_tmd_smem<Q>() ? 6 : 5;
  static constexpr size_t bytes = sizeof(uint32_t) * (size_t)(SROWS + TROWS) * ROWW;
};

// Tensor memory (TMEM) as the transition store.  tcgen05.ld reads ~370 B/clk/SM beside the
// 128 B/clk/SM of LDS, and the two add up (profiles/tmem_bw_r02z.jsonl), so the six transition
// vectors the row streams move off the shared-memory pipe that bounds the shared-memory variant
// (L1/smem 90% busy, profiles/ncu_vit_wide_2048_r02y.md).  Every warp keeps its own copy in its
// 32-lane TMEM quarter (a warp can only address lanes 32 (warp % 4) ..): TMEM lane z of the
// quarter holds lane z's words, 32 columns per chunk of four registers --
// [tMM x4 | tIM x4 | tDM x4 | tMI x4 | tII x4 | tMD x4 | unused x8] -- 256 columns at Q = 32,
// allocated per CTA (a power of two >= 32; the launcher keeps the CTAs per SM within the 512).
template <int Q>
constexpr int wide_tmem_cols() { return Q <= 8 ? 64 : Q <= 16 ? 128 : 256; }

__device__ __forceinline__ void tm_ld16(uint32_t a, uint32_t (&v)[16]) {
  asm volatile("tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
               : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7]),
                 "=r"(v[8]), "=r"(v[9]), "=r"(v[10]), "=r"(v[11]), "=r"(v[12]), "=r"(v[13]), "=r"(v[14]), "=r"(v[15])
               : "r"(a));
}
__device__ __forceinline__ void tm_ld4(uint32_t a, uint32_t (&v)[4]) {
  asm volatile("tcgen05.ld.sync.aligned.32x32b.x4.b32 {%0,%1,%2,%3}, [%4];"
               : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]) : "r"(a));
}
__device__ __forceinline__ void tm_st8(uint32_t a, const uint32_t (&v)[8]) {
  asm volatile("tcgen05.st.sync.aligned.32x32b.x8.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8};"
               ::"r"(a), "r"(v[0]), "r"(v[1]), "r"(v[2]), "r"(v[3]), "r"(v[4]), "r"(v[5]), "r"(v[6]), "r"(v[7])
               : "memory");
}
// tcgen05.wait::ld, threaded through the destination registers of the loads it waits for so that
// no use of them is scheduled above it
__device__ __forceinline__ void tm_wait(uint32_t (&a)[16], uint32_t (&b)[4]) {
  asm volatile("tcgen05.wait::ld.sync.aligned;"
               : "+r"(a[0]), "+r"(a[1]), "+r"(a[2]), "+r"(a[3]), "+r"(a[4]), "+r"(a[5]), "+r"(a[6]), "+r"(a[7]),
                 "+r"(a[8]), "+r"(a[9]), "+r"(a[10]), "+r"(a[11]), "+r"(a[12]), "+r"(a[13]), "+r"(a[14]), "+r"(a[15]),
                 "+r"(b[0]), "+r"(b[1]), "+r"(b[2]), "+r"(b[3])
               :: "memory");
}
__device__ __forceinline__ void tm_wait(uint32_t (&b)[4]) {
  asm volatile("tcgen05.wait::ld.sync.aligned;" : "+r"(b[0]), "+r"(b[1]), "+r"(b[2]), "+r"(b[3]) :: "memory");
}

template <int Q, bool TM>
struct VitWideLane {
  static constexpr int NC = Q / 4;
  static constexpr bool TMD_S = TM || wide_tmd_smem<Q>();
  uint32_t tMD[TMD_S ? 1 : Q], tDD[Q];   // the D chain's transitions (s16x2)
  uint32_t Mc[Q], Ic[Q], Dc[Q], Bk[Q];
  uint32_t R, thrv;
  int F, xJ, move, safe, tbm_min, state;

  __device__ __forceinline__ void load(const uint32_t* __restrict__ tr, int z) {
#pragma unroll
    for (int q = 0; q < Q; ++q) {
      if constexpr (!TMD_S) tMD[q] = tr[4 * 32 * Q + z * Q + q];
      tDD[q] = tr[7 * 32 * Q + z * Q + q];
    }
  }
  __device__ __forceinline__ bool set_bk(const uint32_t* __restrict__ tbm, int z, int xB) {
    bool okv = true;
#pragma unroll
    for (int q = 0; q < Q; ++q) {
      const uint32_t w = __ldg(tbm + z * Q + q);
      const int lo = max(-32768, min(32767, xB + (int)(int16_t)(w & 0xffffu))) - F;
      const int hi = max(-32768, min(32767, xB + (int)(int16_t)(w >> 16))) - F;
      okv = okv && lo <= safe && hi <= safe;
      Bk[q] = (uint32_t)max(lo, 0) | ((uint32_t)max(hi, 0) << 16);
    }
    return okv;
  }
  __device__ __forceinline__ void set_thr(int thr) {
    const int t = min(thr - F, safe + 1);
    thrv = (uint32_t)(0x8000 - t) * 0x10001u;
  }
  __device__ __forceinline__ void kill() {
#pragma unroll
    for (int q = 0; q < Q; ++q) Mc[q] = Ic[q] = Dc[q] = Bk[q] = 0u;
    R = 0u;
    thrv = 0x80008000u;
  }
  __device__ __forceinline__ void rebase(int d, uint32_t& cout) {
    if (d <= 0) return;
    const uint32_t n = d >= 32768 ? 0x80008000u : (uint32_t)(uint16_t)(-d) * 0x10001u;
#pragma unroll
    for (int q = 0; q < Q; ++q) {
      Mc[q] = __viaddmax_s16x2_relu(Mc[q], n, n);
      Ic[q] = __viaddmax_s16x2_relu(Ic[q], n, n);
      Dc[q] = __viaddmax_s16x2_relu(Dc[q], n, n);
    }
    R = __viaddmax_s16x2_relu(R, n, n);
    cout = __viaddmax_s16x2_relu(cout, n, n);
  }
  __device__ __forceinline__ void start(const uint32_t* __restrict__ tbm, int z, int mv, int tmin, int sf) {
#pragma unroll
    for (int q = 0; q < Q; ++q) Mc[q] = Ic[q] = Dc[q] = 0u;   // Alg 2 l.9: -inf -> floor
    R = 0u;
    move = mv;
    tbm_min = tmin;
    F = max(-32768, kBaseW + mv + tmin);
    safe = sf;
    xJ = kNegW;
    state = 0;
    const bool okv = set_bk(tbm, z, kBaseW + move);            // xB = xN + N->B
    if (__any_sync(0xffffffffu, !okv)) state = 2;
    if (state) kill();
    else set_thr(min(kBaseW + 501, 32767));
  }

  // M and I of the four nodes of chunk c, highest first
  __device__ __forceinline__ void mi_chunk(int c, uint4 ev, const uint32_t* tmm, const uint32_t* tim,
                                           const uint32_t* tdm, const uint32_t* tmi, const uint32_t* tii,
                                           uint32_t cM, uint32_t cI, uint32_t cD) {
    const uint32_t e4[4] = {ev.x, ev.y, ev.z, ev.w};
#pragma unroll
    for (int j = 3; j >= 0; --j) {
      const int q = 4 * c + j;
      const uint32_t pm = q ? Mc[q - 1] : cM;
      const uint32_t pi = q ? Ic[q - 1] : cI;
      const uint32_t pd = q ? Dc[q - 1] : cD;
      uint32_t m = __viaddmax_s16x2(pm, tmm[j], Bk[q]);
      m = __viaddmax_s16x2(pi, tim[j], m);
      m = __viaddmax_s16x2(pd, tdm[j], m);
      Ic[q] = __viaddmax_s16x2(Ic[q], tii[j], __viaddmax_s16x2_relu(Mc[q], tmi[j], tmi[j]));
      Mc[q] = __viaddmax_s16x2_relu(m, e4[j], e4[j]);
    }
  }

  // one DP row; er: the residue's emission row (shared or, for rare codes, global; chunk layout),
  // ts_s: shared address of the five transition vectors (chunk layout), or with TM the TMEM
  // address of this warp's quarter
  __device__ __forceinline__ void row(const uint32_t* __restrict__ er, uint32_t ts_s, const uint32_t* __restrict__ tbm,
                                      int z) {
    constexpr int ROWW = Q * 32;
    const uint32_t sel = (z == 0) ? 0x1054u : 0x3210u;   // lane 0: low <- floor, high <- lane 31 low
    const int src = (z + 31) & 31;
    uint32_t cM = __shfl_sync(0xffffffffu, Mc[Q - 1], src);
    uint32_t cI = __shfl_sync(0xffffffffu, Ic[Q - 1], src);
    uint32_t cD = __shfl_sync(0xffffffffu, Dc[Q - 1], src);
    cM = __byte_perm(cM, 0u, sel);
    cI = __byte_perm(cI, 0u, sel);
    cD = __byte_perm(cD, 0u, sel);
    // M and I (Alg 2 l.15-16, emission per reading R15), highest chunk first: q-1 still holds row i-1
    if constexpr (TM) {
      // transitions from TMEM, one chunk ahead: wait::ld for chunk c, issue chunk c - 1, compute c
      uint32_t ta[2][16], tb[2][4];
      tm_ld16(ts_s + (uint32_t)((NC - 1) * 32), ta[(NC - 1) & 1]);
      tm_ld4(ts_s + (uint32_t)((NC - 1) * 32 + 16), tb[(NC - 1) & 1]);
#pragma unroll
      for (int c = NC - 1; c >= 0; --c) {
        const uint32_t off = (uint32_t)(c * 4 * 32 + z * 4);
        const uint4 ev = *reinterpret_cast<const uint4*>(er + off);
        tm_wait(ta[c & 1], tb[c & 1]);
        if (c > 0) {
          tm_ld16(ts_s + (uint32_t)((c - 1) * 32), ta[(c - 1) & 1]);
          tm_ld4(ts_s + (uint32_t)((c - 1) * 32 + 16), tb[(c - 1) & 1]);
        }
        const uint32_t* t = ta[c & 1];
        mi_chunk(c, ev, t, t + 4, t + 8, t + 12, tb[c & 1], cM, cI, cD);
      }
    } else {
#pragma unroll
      for (int c = NC - 1; c >= 0; --c) {
        const uint32_t off = (uint32_t)(c * 4 * 32 + z * 4);
        const uint4 ev = *reinterpret_cast<const uint4*>(er + off);
        uint4 tv[5];
#pragma unroll
        for (int v = 0; v < 5; ++v) tv[v] = lds4<(Q > 20)>(ts_s + (uint32_t)(v * ROWW + off) * 4u);
        const uint32_t tmm[4] = {tv[0].x, tv[0].y, tv[0].z, tv[0].w};
        const uint32_t tim[4] = {tv[1].x, tv[1].y, tv[1].z, tv[1].w};
        const uint32_t tdm[4] = {tv[2].x, tv[2].y, tv[2].z, tv[2].w};
        const uint32_t tmi[4] = {tv[3].x, tv[3].y, tv[3].z, tv[3].w};
        const uint32_t tii[4] = {tv[4].x, tv[4].y, tv[4].z, tv[4].w};
        mi_chunk(c, ev, tmm, tim, tdm, tmi, tii, cM, cI, cD);
      }
    }
#pragma unroll
    for (int q = 0; q + 1 < Q; q += 2) R = __vimax3_s16x2(R, Mc[q], Mc[q + 1]);
    // D: partial from M (l.17, reading R16) fused with the in-lane D->D chain
    uint32_t cout;
    if constexpr (TMD_S) {
      uint32_t prev = 0u;                      // D of the previous node (node 0 of the lane: floor)
      uint4 tn;                                // tMD chunk c + 1, one ahead
      uint32_t tq[2][4];                       // (TMEM: chunk c + 1 in flight)
      if constexpr (TM) tm_ld4(ts_s + 20u, tq[0]);
      else tn = lds4<true>(ts_s + (uint32_t)(5 * ROWW + z * 4) * 4u);
#pragma unroll
      for (int c = 0; c < NC; ++c) {
        uint32_t tmd[4];
        if constexpr (TM) {
          tm_wait(tq[c & 1]);
          if (c + 1 < NC) tm_ld4(ts_s + (uint32_t)((c + 1) * 32 + 20), tq[(c + 1) & 1]);
#pragma unroll
          for (int j = 0; j < 4; ++j) tmd[j] = tq[c & 1][j];
        } else {
          const uint4 tv = tn;
          if (c + 1 < NC) tn = lds4<true>(ts_s + (uint32_t)(5 * ROWW + (c + 1) * 4 * 32 + z * 4) * 4u);
          tmd[0] = tv.x;
          tmd[1] = tv.y;
          tmd[2] = tv.z;
          tmd[3] = tv.w;
        }
#pragma unroll
        for (int j = 0; j < 4; ++j) {
          const int q = 4 * c + j;
          Dc[q] = q ? prev : 0u;
          prev = __viaddmax_s16x2(Dc[q], tDD[q], __viaddmax_s16x2_relu(Mc[q], tmd[j], tmd[j]));
        }
      }
      cout = prev;
    } else {
      Dc[0] = 0u;
#pragma unroll
      for (int q = 1; q < Q; ++q)
        Dc[q] = __viaddmax_s16x2(Dc[q - 1], tDD[q - 1], __viaddmax_s16x2_relu(Mc[q - 1], tMD[q - 1], tMD[q - 1]));
      cout = __viaddmax_s16x2(Dc[Q - 1], tDD[Q - 1], __viaddmax_s16x2_relu(Mc[Q - 1], tMD[Q - 1], tMD[Q - 1]));
    }
    // hit / overflow / safe-bound vote (Alg 2 l.22-24 on the rows that need it)
    const bool hit = (__vadd2(R, thrv) & 0x80008000u) != 0u;
    if (__any_sync(0xffffffffu, hit)) {
      uint32_t mm = R;
#pragma unroll
      for (int o = 16; o >= 1; o >>= 1) mm = __vmaxs2(mm, __shfl_xor_sync(0xffffffffu, mm, o));
      const int mp = max((int)(mm & 0xffffu), (int)(mm >> 16));
      bool okv = true;
      if (state == 0) {
        if (mp > safe) {
          state = 2;                                  // beyond the 16-bit window: s32 re-score
        } else if (mp + F >= 32767) {
          state = 1;                                  // reading R17: overflow -> +inf, pass
        } else {
          xJ = mp + F - 500;                          // E->J (and E->C: xC == xJ)
          const int xB = max(xJ, kBaseW) + move;
          const int Fn = max(-32768, min(32767, xB + tbm_min));
          rebase(Fn - F, cout);
          F = Fn;
          okv = set_bk(tbm, z, xB);
          set_thr(min(max(xJ, kBaseW) + 501, 32767));
        }
      }
      if (__any_sync(0xffffffffu, !okv) && state == 0) state = 2;
      if (state) kill();
    }
    // Lazy-F across the 64 virtual lanes (l.25, Fig 7): passes while any carry improves (R19)
    for (;;) {
      uint32_t cin = __shfl_sync(0xffffffffu, cout, src);
      cin = __byte_perm(cin, 0u, sel);
      bool imp = __vmaxs2(cin, Dc[0]) != Dc[0];
      if (!__any_sync(0xffffffffu, imp)) break;
      Dc[0] = __vmaxs2(Dc[0], cin);
      constexpr int K0 = 3;                  // most D->D runs die within a few nodes
#pragma unroll
      for (int q = 1; q < K0; ++q) {
        const uint32_t nd = __viaddmax_s16x2_relu(Dc[q - 1], tDD[q - 1], tDD[q - 1]);
        imp = imp && (__vmaxs2(nd, Dc[q]) != Dc[q]);
        Dc[q] = __vmaxs2(Dc[q], nd);
      }
      if (__any_sync(0xffffffffu, imp)) {
#pragma unroll
        for (int q = K0; q < Q; ++q) Dc[q] = __viaddmax_s16x2(Dc[q - 1], tDD[q - 1], Dc[q]);
        cout = __viaddmax_s16x2(Dc[Q - 1], tDD[Q - 1], cout);
      } else {
        break;
      }
    }
  }

  __device__ __forceinline__ int finish() {
    uint32_t mm = R;
#pragma unroll
    for (int o = 16; o >= 1; o >>= 1) mm = __vmaxs2(mm, __shfl_xor_sync(0xffffffffu, mm, o));
    const int mp = max((int)(mm & 0xffffu), (int)(mm >> 16));
    if (state == 1) return 32767;
    if (state == 2) return kRedo;
    if (mp > 0) return max(xJ, max(kNegW, mp + F - 500));
    return xJ > kNegW ? xJ : kRedo;
  }
};

// threads per CTA: the TMEM variant runs one CTA of eight warps per SM (warps w and w + 4 read the
// same lane quarter), the shared-memory one two CTAs of four
template <bool TM> constexpr int wide_threads() { return TM ? 256 : 128; }

template <int Q, bool TM>
__global__ void __launch_bounds__(wide_threads<TM>(), TM ? 1 : 2) vit_wide_kernel(const VitArgs a) {
  using S = VitWideSmem<Q, TM>;
  constexpr int ROWW = S::ROWW;
  extern __shared__ uint4 smem4[];
  uint32_t* sm = reinterpret_cast<uint32_t*>(smem4);
  const uint32_t* tr = reinterpret_cast<const uint32_t*>(a.tr);
  {
    const uint4* src = reinterpret_cast<const uint4*>(a.rsc);
    constexpr int R16 = ROWW / 4;
    for (int i = threadIdx.x; i < 20 * R16; i += blockDim.x) smem4[i] = src[i];
    for (int i = threadIdx.x; i < R16; i += blockDim.x) smem4[20 * R16 + i] = src[26 * R16 + i];
    // tMM, tIM, tDM, tMI, tII ([8][32][Q] plain) into the chunk layout: word q of lane z at
    // (q / 4) * 128 + z * 4 + q % 4
    const int vsel[6] = {1, 2, 3, 5, 6, 4};
    for (int i = threadIdx.x; i < S::TROWS * ROWW; i += blockDim.x) {
      const int v = i / ROWW, o = i - v * ROWW, z = o / Q, q = o - z * Q;
      sm[(S::SROWS + v) * ROWW + (q >> 2) * 128 + z * 4 + (q & 3)] = tr[vsel[v] * ROWW + o];
    }
  }
  const int lane = threadIdx.x & 31;
  __shared__ uint32_t tmem_base;
  uint32_t ts_s;
  if constexpr (TM) {
    if (threadIdx.x < 32) {
      asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;"
                   ::"r"((uint32_t)__cvta_generic_to_shared(&tmem_base)), "n"(wide_tmem_cols<Q>()));
      asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    asm volatile("tcgen05.fence::before_thread_sync;");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;");
    ts_s = tmem_base + ((uint32_t)(threadIdx.x & 96) << 16);   // this warp's lane quarter
    // this lane's words, chunk by chunk ([8][32][Q] plain rows of tr: 1 tMM, 2 tIM, 3 tDM, 5 tMI,
    // 6 tII, 4 tMD)
    constexpr int vsel[6] = {1, 2, 3, 5, 6, 4};
    if (threadIdx.x < 128) {                  // warps 0-3 fill the four quarters
#pragma unroll 1
      for (int c = 0; c < Q / 4; ++c) {
#pragma unroll
        for (int h = 0; h < 3; ++h) {
          uint32_t v[8];
#pragma unroll
          for (int j = 0; j < 8; ++j) v[j] = tr[vsel[2 * h + j / 4] * ROWW + lane * Q + 4 * c + (j & 3)];
          tm_st8(ts_s + (uint32_t)(c * 32 + 8 * h), v);
        }
      }
      asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
    }
    asm volatile("tcgen05.fence::before_thread_sync;");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;");
  } else {
    __syncthreads();
    ts_s = (uint32_t)__cvta_generic_to_shared(sm + S::SROWS * ROWW);
  }
  const uint32_t* rare = reinterpret_cast<const uint32_t*>(a.rsc);
  VitWideLane<Q, TM> V;
  V.load(tr, lane);
  const long long ntot = a.list ? *a.nlist : a.nseq;
  for (;;) {
    unsigned long long b = 0;
    if (lane == 0) b = atomicAdd(a.counter, 1ull);
    b = __shfl_sync(0xffffffffu, b, 0);
    if ((long long)b >= ntot) break;
    const int s = a.list ? a.list[b] : (int)b;
    if (s < a.ndone && a.done[s]) continue;
    const int L = a.len[s];
    const uint32_t* wp = a.words + (size_t)a.woff16[s] * 4;
    V.start(tr, lane, a.move[L], a.tbm_min, a.safe);
    ResStream rs;
    rs.init(wp, (L + 5) / 6);
    for (int iq = 0; iq < rs.nq && V.state == 0; ++iq) {
      uint4 w4 = rs.next(iq);
#pragma unroll 1
      for (int k = 0; k < 4; ++k) {
        const uint32_t w = w4.x;
        w4.x = w4.y;
        w4.y = w4.z;
        w4.z = w4.w;
#pragma unroll 1
        for (int j = 0; j < 6; ++j) {
          const int x = (w >> (5 * j)) & 31;
          if (x == 31) break;                      // pad slots
          const uint32_t* er = (x < 20 || x == 26) ? sm + (x < 20 ? x : 20) * ROWW : rare + x * ROWW;
          V.row(er, ts_s, tr, lane);
        }
      }
    }
    const int raw = V.finish();
    if (lane == 0) {
      if (raw >= -32768) {
        a.raw_sorted[s] = (int16_t)raw;
      } else {
        const unsigned long long k = atomicAdd(a.redo_count, 1ull);
        a.redo_list[k] = s;
      }
    }
  }
  if constexpr (TM) {
    asm volatile("tcgen05.fence::before_thread_sync;");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;");
    if (threadIdx.x < 32)
      asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem_base), "n"(wide_tmem_cols<Q>()));
  }
}

}  // namespace hmg
