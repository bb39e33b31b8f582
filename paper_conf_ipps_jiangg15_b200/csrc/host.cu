// host.cu -- libhmg host side: quantiser, DB packer/sorter, threshold tables,
// kernel geometry policy and the C ABI declared in include/hmg.h.
//
// The quantiser implements HMMER 3.0's byte and word score systems (the
// paper: "8-bit saturating scoring system"; "bias", Alg 1 l.15
// P:638; "-32768" word -inf, Alg 2 l.9 P:674; constants per DESIGN.md R1-R10).
// It is written independently of oracle/ (no shared code); tests require the
// two to agree byte-for-byte.
#include <cuda_runtime.h>

#include <algorithm>
#include <cmath>
#include <cstdlib>
#include <cstring>
#include <map>
#include <mutex>
#include <new>
#include <numeric>
#include <random>
#include <string>
#include <vector>

#include "hmg_internal.h"

using namespace hmg;

std::atomic<long long> hmg::g_launches{0};

namespace {

// ---------------------------------------------------------------- stage timing (profiling aid)
// Stages: 0 MSV fast kernel | 1 MSV exact redo (select + kernel) | 2 MSV flags + compaction |
//         3 Viterbi kernel | 4 Viterbi flags/scatter | 5 Viterbi-pass compaction + Forward kernel.  Marks are CUDA events on the call's stream.
constexpr int kStages = 6;
struct StageTimer {
  bool on = false;
  int device = -1;
  cudaEvent_t ev[kStages + 1] = {};
  bool rec[kStages + 1] = {};
  unsigned long long* h_redo = nullptr;   // pinned: sequences the pair Viterbi kernel handed back
  bool redo_rec = false;
} g_timer;
std::mutex g_timer_mu;

void mark(int i, cudaStream_t st) {
  if (!g_timer.on) return;
  if (cudaEventRecord(g_timer.ev[i], st) == cudaSuccess) g_timer.rec[i] = true;
}
void mark_reset() {
  if (!g_timer.on) return;
  for (bool& r : g_timer.rec) r = false;
  g_timer.redo_rec = false;
}
void stage_count_redo(const unsigned long long* d, cudaStream_t st) {
  if (!g_timer.on || !g_timer.h_redo) return;
  if (cudaMemcpyAsync(g_timer.h_redo, d, sizeof(unsigned long long), cudaMemcpyDeviceToHost, st) == cudaSuccess)
    g_timer.redo_rec = true;
}

constexpr double kLn2 = 0.693147180559945309417232121458176568;
constexpr float kFwdMscMax = 40.0f;   // Forward odds space: emission log-odds above this could overflow float

// ---------------------------------------------------------------- quantisation
struct Scales {
  float b = (float)(3.0 / kLn2);    // third-bits (R1)
  float w = (float)(500.0 / kLn2);  // 1/500 bits (R2)
};

// unbiased byte cost of a non-positive score, capped at 255 (R3)
int cost_unbiased(float sc, const Scales& S) {
  const float c = -roundf(S.b * sc);
  return c > 255.0f ? 255 : (int)c;
}

// biased byte cost; 255 is -inf (R4)
uint8_t cost_biased(float sc, int bias, const Scales& S) {
  const float c = -roundf(S.b * sc);
  if (c > (float)(255 - bias)) return 255;
  const int v = (int)c + bias;
  return (uint8_t)(v < 0 ? 0 : v);
}

// word score clamped to int16 (R5)
int16_t word(float sc, const Scales& S) {
  const float r = roundf(S.w * sc);
  if (r >= 32767.0f) return 32767;
  if (r <= -32768.0f) return -32768;
  return (int16_t)r;
}

int tjb_of(int L) { return cost_unbiased(logf(3.0f / (float)(L + 3)), Scales()); }  // R10
int16_t move_of(int L) { return word(logf(3.0f / (float)(L + 3)), Scales()); }      // R10

// ---------------------------------------------------------------- statistics (R11, R24, R25)
float msv_nats_of(int raw, int L) {
  if (raw == 255) return INFINITY;
  const Scales S;
  float v = (float)(raw - tjb_of(L)) - (float)kBaseB;
  v /= S.b;
  v -= 3.0;
  return v;
}

float vit_nats_of(int raw, int L) {
  if (raw == 32767) return INFINITY;
  if (raw == -32768) return -INFINITY;
  const Scales S;
  float v = (float)(raw + move_of(L)) - (float)kBaseW;
  v /= S.w;
  v -= 3.0;
  return v;
}

float null1_of(int L) {
  const float p1 = (float)L / (float)(L + 1);
  return (float)((float)L * log((double)p1) + log(1.0 - (double)p1));
}

double gumbel_surv(double x, double mu, double lambda) {
  const double y = lambda * (x - mu);
  const double ey = -exp(-y);
  return fabs(ey) < 5e-9 ? -ey : 1.0 - exp(ey);
}

bool passes(float nats, int L, double mu, double lambda, double F) {
  double P;
  if (nats == INFINITY) P = 0.0;
  else if (nats == -INFINITY) P = 1.0;
  else P = gumbel_surv((double)(nats - null1_of(L)) / kLn2, mu, lambda);
  return !(P > F);
}

// least raw in [lo, hi] that passes (pass is monotone in raw), hi+1 if none
template <class Pass>
int least_passing(int lo, int hi, Pass pass) {
  if (!pass(hi)) return hi + 1;
  while (lo < hi) {
    const int mid = lo + (hi - lo) / 2;
    if (pass(mid)) hi = mid;
    else lo = mid + 1;
  }
  return lo;
}

// ---------------------------------------------------------------- helpers
struct Dev {
  int saved = -1;
  explicit Dev(int d) {
    cudaGetDevice(&saved);
    if (saved != d) cudaSetDevice(d);
  }
  ~Dev() {
    int cur = -1;
    cudaGetDevice(&cur);
    if (saved >= 0 && cur != saved) cudaSetDevice(saved);
  }
};

hmg_status cuda_status(cudaError_t e) {
  if (e == cudaSuccess) return HMG_OK;
  cudaGetLastError();
  return e == cudaErrorMemoryAllocation ? HMG_ENOMEM : HMG_ECUDA;
}

template <class T>
hmg_status upload(T** d, const T* h, size_t n) {
  *d = nullptr;
  if (n == 0) n = 1;
  cudaError_t e = cudaMalloc(reinterpret_cast<void**>(d), n * sizeof(T));
  if (e != cudaSuccess) return cuda_status(e);
  if (h) e = cudaMemcpy(*d, h, n * sizeof(T), cudaMemcpyHostToDevice);
  return cuda_status(e);
}

// Tuning / debug overrides (hmg_set_tuning): the library never reads the process environment.
// Knob names are the kernel-geometry and schedule choices of DESIGN.md; an unset knob takes the
// measured default at its call site.
const char* const kTuneNames[] = {
    "MSV_G", "VIT_G", "MSV_LLONG", "NO_LONG_LANE", "FWD_QMAX", "FWD_W", "FWD_S", "VIT_CTA", "VIT_CTA_W",
    "VIT_GENERIC", "NO_VIT_PAIR", "VIT_PAIR_G", "VIT_PAIR_CTA", "VIT_SCAN", "VIT_PAIR_W", "VIT_PAIR_SG",
    "VIT_CPAIR2", "LONG_S32", "PIPE_LLONG", "PIPE_CHUNK", "UPLOAD_PARTS", "UPLOAD_FIRST_PERMILLE",
    "UPLOAD_GROW", "PIPE_LONG_SMS", "MSV_BATCH_PAD", "MSV_BATCH_ROUNDS", "VIT_WIDE", "LONG_PAIR_SMALL",
    "UPLOAD_MSV_STREAMS"};
std::mutex g_tune_mu;
std::map<std::string, int> g_tune;

bool tune_known(const char* name) {
  for (const char* k : kTuneNames)
    if (!strcmp(k, name)) return true;
  return false;
}

int tune_int(const char* name, int dflt) {
  std::lock_guard<std::mutex> g(g_tune_mu);
  auto it = g_tune.find(name);
  return it == g_tune.end() ? dflt : it->second;
}

// Stream-ordered scratch (Scratch below) comes from the device's default memory pool; its default
// release threshold (0) returns the memory to the driver at every synchronisation, so each eager
// call would map its scratch again (milliseconds for the DB-sized buffers).  Keep it cached.
void keep_pool_cached(int device) {
  static std::mutex mu;
  static std::vector<bool> done;
  std::lock_guard<std::mutex> g(mu);
  if ((int)done.size() <= device) done.resize(device + 1, false);
  if (done[device]) return;
  cudaMemPool_t pool = nullptr;
  if (cudaDeviceGetDefaultMemPool(&pool, device) == cudaSuccess) {
    uint64_t thr = UINT64_MAX;
    cudaMemPoolSetAttribute(pool, cudaMemPoolAttrReleaseThreshold, &thr);
  }
  cudaGetLastError();
  done[device] = true;
}

// ---------------------------------------------------------------- kernel geometry
void msv_geometry(int M, int* G, int* Q) {
  // lane-group size from the G sweep on the config-2 DB (profiles/msv_sweep_r01.txt)
  int g = M < 80 ? 4 : M <= 450 ? 8 : M <= 640 ? 16 : 32;
  const int o = tune_int("MSV_G", 0);
  if (o == 4 || o == 8 || o == 16 || o == 32) g = o;
  // 2GQ >= M: the fast kernel records each cell's value in the cell it feeds (t_{i+1}[k+1]); node
  // M's, which no cell receives when 2GQ = M, enters the running max through the outgoing carry
  // (msv.cuh).  (MSV_Q_PLUS1 builds: 2GQ >= M + 1, a padding successor cell.)
  const int extra = kMsvQPlus1 ? 1 : 0;
  int q = (M + extra + 2 * g - 1) / (2 * g);
  while (q > msv_q_max(g) && g < 32) {
    g *= 2;
    q = (M + extra + 2 * g - 1) / (2 * g);
  }
  *G = g;
  *Q = q <= msv_q_max(g) ? q : 0;   // 0: no register kernel, exact kernel only
}

void vit_geometry(int M, int* G, int* Q) {
  int g = M <= 128 ? 8 : M <= 256 ? 16 : 32;
  const int o = tune_int("VIT_G", 0);
  if (o == 8 || o == 16 || o == 32) g = o;
  int q = (M + g - 1) / g;
  while (q > vit_q_max(g) && g < 32) {
    g *= 2;
    q = (M + g - 1) / g;
  }
  *G = g;
  *Q = q <= vit_q_max(g) ? q : 0;
}

// striped MSV table: row x, register q of lane z holds e for nodes z*Q+q+1 (lo), (z+G)*Q+q+1 (hi),
// in the layout of MsvLayout<G, Q> (msv.cuh): 4-word chunks, then the 2-word and 1-word remainder
// chunks in L.nc2 / L.nc1 per-group copies; G < 8: L.ncopy whole-table copies, rows padded to
// 128 B, copy k shifted 16*G*k B
std::vector<uint32_t> msv_table(const hmg_profile& p, int G, int Q) {
  const int M = p.M;
  const MsvLayoutRT L(G, Q);
  auto e_of = [&](int x, int node) -> int16_t {   // node 1-based
    if (x >= kAlpha || node > M) return kNegE;
    return (int16_t)(p.bias - (int)p.cost[(size_t)x * M + (node - 1)]);
  };
  std::vector<uint32_t> out((size_t)L.words, 0u);
  for (int k = 0; k < L.ncopy; ++k)
    for (int x = 0; x < kRows; ++x) {
      uint32_t* row = out.data() + (size_t)k * (L.copy + 4 * G) + (size_t)x * L.stride;
      for (int z = 0; z < G; ++z)
        for (int q = 0; q < Q; ++q) {
          const uint16_t lo = (uint16_t)e_of(x, z * Q + q + 1);
          const uint16_t hi = (uint16_t)e_of(x, (z + G) * Q + q + 1);
          const uint32_t v = (uint32_t)lo | ((uint32_t)hi << 16);
          auto b8 = [](int16_t x) { return (uint32_t)(uint8_t)(int8_t)std::max<int>(x, -128); };
          if (q < L.n4 * 4) {
            row[(q / 4) * 4 * G + z * 4 + (q % 4)] = v;
          } else if (L.byte && q < L.n4 * 4 + 2) {    // int8 pair: bytes 2 (q - 4 n4) (lo, hi)
            const int sh = 16 * (q - L.n4 * 4);
            for (int j = 0; j < 32 / G; ++j) {
              uint32_t& w = row[L.b2 + j * G + z];
              w |= (b8((int16_t)lo) | (b8((int16_t)hi) << 8)) << sh;
            }
          } else if (L.has2 && q < L.n4 * 4 + 2) {
            for (int j = 0; j < L.nc2; ++j) row[L.b2 + j * 2 * G + z * 2 + (q - L.n4 * 4)] = v;
          } else {
            for (int j = 0; j < L.nc1; ++j) row[L.b1 + j * G + z] = v;
          }
        }
    }
  return out;
}

// Viterbi register-kernel tables: emissions as s32 in the MSV chunk layout over Q words per lane
// (lane z: nodes z*Q+1..z*Q+Q), transitions as s32 [8][G*Q] with node (z*Q+q+1) at z*Q+q;
// nodes > M are -inf.
void vit_tables(const hmg_profile& p, int G, int Q, std::vector<uint32_t>* rsc, std::vector<int32_t>* tr) {
  const int M = p.M;
  const int ROWW = Q * G;
  rsc->assign(((size_t)kRows * ROWW + 3) / 4 * 4, 0);
  const int n4 = Q / 4, r = Q % 4;
  auto word_index = [&](int z, int q) {
    if (q < n4 * 4) return (q / 4) * 4 * G + z * 4 + (q % 4);
    int b = n4 * 4 * G;
    int qq = q - n4 * 4;
    if (r >= 2) {
      if (qq < 2) return b + z * 2 + qq;
      b += 2 * G;
      qq -= 2;
    }
    return b + z;
  };
  for (int x = 0; x < kRows; ++x)
    for (int z = 0; z < G; ++z)
      for (int q = 0; q < Q; ++q) {
        const int node = z * Q + q + 1;
        const int v = (x >= kAlpha || node > M) ? kNegW : (int)p.rsc[(size_t)x * M + node - 1];
        (*rsc)[(size_t)x * ROWW + word_index(z, q)] = (uint32_t)v;
      }
  tr->assign((size_t)8 * G * Q, kNegW);
  for (int t = 0; t < 8; ++t)
    for (int o = 0; o < G * Q; ++o)
      if (o < M) (*tr)[(size_t)t * G * Q + o] = p.tsc[(size_t)t * M + o];
}

// block-per-sequence kernel tables: emissions as s16 pairs (node g*Q+2h+1 low, +2 high) in the
// chunk layout over Q/2 words per lane; transitions as vit_tables.
void vit_tables_s16(const hmg_profile& p, int NT, int Q, std::vector<uint32_t>* rsc, std::vector<int32_t>* tr) {
  const int M = p.M;
  const int Q2 = Q / 2;
  const int ROWW = Q2 * NT;
  rsc->assign((size_t)kRows * ROWW, 0);
  const int n4 = Q2 / 4, r = Q2 % 4;
  auto word_index = [&](int z, int q) {
    if (q < n4 * 4) return (q / 4) * 4 * NT + z * 4 + (q % 4);
    int b = n4 * 4 * NT;
    int qq = q - n4 * 4;
    if (r >= 2) {
      if (qq < 2) return b + z * 2 + qq;
      b += 2 * NT;
      qq -= 2;
    }
    return b + z;
  };
  auto r_of = [&](int x, int node) -> uint16_t {
    if (x >= kAlpha || node > M) return (uint16_t)(int16_t)kNegW;
    return (uint16_t)p.rsc[(size_t)x * M + node - 1];
  };
  for (int x = 0; x < kRows; ++x)
    for (int z = 0; z < NT; ++z)
      for (int h = 0; h < Q2; ++h)
        (*rsc)[(size_t)x * ROWW + word_index(z, h)] =
            (uint32_t)r_of(x, z * Q + 2 * h + 1) | ((uint32_t)r_of(x, z * Q + 2 * h + 2) << 16);
  tr->assign((size_t)8 * NT * Q, kNegW);
  for (int t = 0; t < 8; ++t)
    for (int o = 0; o < NT * Q; ++o)
      if (o < M) (*tr)[(size_t)t * NT * Q + o] = p.tsc[(size_t)t * M + o];
}

// pair-kernel tables (vit_pair.cuh): register q of lane z holds node z*Q+q+1 (low half) and
// (z+G)*Q+q+1 (high half); emissions in the MSV chunk layout over Q words per lane, transitions
// [8][G][Q]; padding nodes and nonexistent transitions are -32768 (the kernel's floor).
void vit_pair_tables(const hmg_profile& p, int G, int Q, std::vector<uint32_t>* rsc, std::vector<uint32_t>* tr) {
  const int M = p.M;
  const int ROWW = Q * G;
  rsc->assign(((size_t)kRows * ROWW + 3) / 4 * 4, 0u);
  const int n4 = Q / 4, r = Q % 4;
  auto word_index = [&](int z, int q) {
    if (q < n4 * 4) return (q / 4) * 4 * G + z * 4 + (q % 4);
    int b = n4 * 4 * G;
    int qq = q - n4 * 4;
    if (r >= 2) {
      if (qq < 2) return b + z * 2 + qq;
      b += 2 * G;
      qq -= 2;
    }
    return b + z;
  };
  auto r_of = [&](int x, int node) -> uint32_t {   // node 1-based
    if (x >= kAlpha || node > M) return (uint16_t)(int16_t)kNegW;
    return (uint16_t)p.rsc[(size_t)x * M + node - 1];
  };
  for (int x = 0; x < kRows; ++x)
    for (int z = 0; z < G; ++z)
      for (int q = 0; q < Q; ++q)
        (*rsc)[(size_t)x * ROWW + word_index(z, q)] = r_of(x, z * Q + q + 1) | (r_of(x, (z + G) * Q + q + 1) << 16);
  auto t_of = [&](int t, int node) -> uint32_t {
    if (node > M) return (uint16_t)(int16_t)kNegW;
    return (uint16_t)p.tsc[(size_t)t * M + node - 1];
  };
  tr->assign((size_t)8 * G * Q, 0u);
  for (int t = 0; t < 8; ++t)
    for (int z = 0; z < G; ++z)
      for (int q = 0; q < Q; ++q)
        (*tr)[(size_t)t * G * Q + z * Q + q] = t_of(t, z * Q + q + 1) | (t_of(t, (z + G) * Q + q + 1) << 16);
}

struct Scratch {
  std::vector<void*> bufs;
  cudaStream_t st;
  explicit Scratch(cudaStream_t s) : st(s) {}
  void* get(size_t n, cudaError_t* err) {
    void* p = nullptr;
    cudaError_t e = cudaMallocAsync(&p, n ? n : 16, st);
    if (e != cudaSuccess) {
      *err = e;
      return nullptr;
    }
    bufs.push_back(p);
    return p;
  }
  ~Scratch() {
    for (void* p : bufs) cudaFreeAsync(p, st);
  }
};

// threshold tables, per (F, length range) in the profile; a table is never freed or replaced
// while the profile lives (graphs and concurrent streams may hold its pointer).  Building one
// (host binary search + cudaMalloc / cudaMemcpy) is not allowed under stream capture: a call being
// captured finds its tables prepared (hmg_prepare_thresholds or an eager call) or fails with
// HMG_EUNSUPPORTED without touching the capture.
template <class T, class Fill>
hmg_status thr_table(hmg_profile* p, std::vector<hmg_profile::Thr>& cache, int Lmax, double F, cudaStream_t st,
                     Fill fill, const T** out) {
  std::lock_guard<std::mutex> g(p->mu);
  for (const auto& c : cache)
    if (c.F == F && c.Lmax >= Lmax) {
      *out = (const T*)c.d;
      return HMG_OK;
    }
  cudaStreamCaptureStatus cs = cudaStreamCaptureStatusNone;
  if (st && cudaStreamIsCapturing(st, &cs) == cudaSuccess && cs != cudaStreamCaptureStatusNone)
    return HMG_EUNSUPPORTED;
  cudaGetLastError();
  const int L1 = std::max(Lmax, 40000);            // one table covers every protein length seen so far
  std::vector<T> h((size_t)L1 + 1);
  fill(h, L1);
  T* d = nullptr;
  hmg_status s = upload(&d, h.data(), h.size());
  if (s != HMG_OK) return s;
  cache.push_back({F, L1, d});
  *out = d;
  return HMG_OK;
}

hmg_status msv_thr_table(hmg_profile* p, const hmg_db* db, double F, const uint16_t** out, cudaStream_t st = nullptr,
                         int Lmax = -1) {
  const double mu = p->ev.mu_msv, lam = p->ev.lambda_msv;
  return thr_table<uint16_t>(p, p->thr_msv, Lmax >= 0 ? Lmax : db->Lmax, F, st, [&](std::vector<uint16_t>& h, int L1) {
    h[0] = 256;
    for (int L = 1; L <= L1; ++L)
      h[L] = (uint16_t)least_passing(0, 254, [&](int r) { return passes(msv_nats_of(r, L), L, mu, lam, F); });
  }, out);
}

hmg_status vit_thr_table(hmg_profile* p, const hmg_db* db, double F, const int32_t** out, cudaStream_t st = nullptr,
                         int Lmax = -1) {
  const double mu = p->ev.mu_vit, lam = p->ev.lambda_vit;
  return thr_table<int32_t>(p, p->thr_vit, Lmax >= 0 ? Lmax : db->Lmax, F, st, [&](std::vector<int32_t>& h, int L1) {
    h[0] = 32767;
    for (int L = 1; L <= L1; ++L)
      h[L] = least_passing(-32768, 32766, [&](int r) { return passes(vit_nats_of(r, L), L, mu, lam, F); });
  }, out);
}

// the fast MSV kernel scores this profile over this DB: its precondition (bias < 66 + tbm, set at
// profile creation) and, for a geometry with the int8 remainder chunk, msv_byte_exact at the DB's
// longest sequence; otherwise the exact kernel scores every sequence
bool msv_fast_on(const hmg_profile* p, const hmg_db* db) {
  if (!p->msv_fast || p->msv_Q <= 0) return false;
  return !MsvLayoutRT(p->msv_G, p->msv_Q).byte || msv_byte_exact(tjb_of(std::max(db->Lmax, 0)), p->tbm, p->bias);
}

MsvArgs msv_args(const hmg_profile* p, const hmg_db* db) {
  MsvArgs a{};
  a.words = db->d_words;
  a.woff16 = db->d_woff16;
  a.len = db->d_len;
  a.nseq = db->nseq;
  a.tjb = db->d_tjb;
  a.prof = p->d_msv_prof;
  a.cost = p->d_cost;
  a.M = p->M;
  a.bias = p->bias;
  a.tbm = p->tbm;
  return a;
}

// number of leading (longest) sorted sequences with L > llong
int64_t count_longer(const hmg_db* db, int llong) {
  const auto it = std::upper_bound(db->len_sorted.begin(), db->len_sorted.end(), llong,
                                   [](int v, int L) { return v > L; });
  return (int64_t)(it - db->len_sorted.begin());
}

double mean_len(const hmg_db* db) { return db->nseq ? (double)db->residues / (double)db->nseq : 0.0; }

// MSV fast kernel over the DB into raw_sorted (device, sorted order).  pipe_nlong >= 0: the
// first pipe_nlong sequences are scored by the pipeline long lane instead.
hmg_status run_msv_fast(const hmg_profile* p, const hmg_db* db, cudaStream_t st, uint8_t* raw_sorted, Scratch& S,
                        int64_t pipe_nlong, bool pdl = false, bool mark0 = true,
                        unsigned long long* ctr_zeroed = nullptr, int64_t end = -1) {
  cudaError_t e = cudaSuccess;
  const int64_t n = db->nseq;
  MsvArgs a = msv_args(p, db);
  a.raw = raw_sorted;
  if (end >= 0) a.nseq = end;          // sorted range [pipe_nlong, end) only (overlapped upload)
  if (pipe_nlong >= 0) {
    a.nlong = pipe_nlong;
    a.skip_long = 1;
  } else {  // in-kernel whole-warp queue: L > max(1000, 8 x mean length) (env HMG_MSV_LLONG)
    a.nlong = count_longer(db, tune_int("MSV_LLONG", (int)std::max(1000.0, 8.0 * mean_len(db))));
    a.skip_long = 0;
  }
  // (with pdl the counters must be zeroed before the preceding kernel: any stream operation
  //  between it and this launch would serialise them)
  auto* ctr = ctr_zeroed;
  if (!ctr) {
    ctr = (unsigned long long*)S.get(sizeof(unsigned long long) * 2, &e);
    if (e) return cuda_status(e);
    if ((e = cudaMemsetAsync(ctr, 0, sizeof(unsigned long long) * 2, st))) return cuda_status(e);
  }
  a.counter = ctr;
  const int nwarps_exact = 148 * 16;
  if (msv_fast_on(p, db)) {
    int ok = 0;
    if (mark0) mark(0, st);
    if ((e = launch_msv_fast(p->msv_G, p->msv_Q, a, st, &ok, pdl))) return cuda_status(e);
    if (!ok) return HMG_EUNSUPPORTED;
    mark(1, st);
  } else {
    auto* scr = (uint8_t*)S.get((size_t)nwarps_exact * 2 * (p->M + 1), &e);
    if (e) return cuda_status(e);
    a.list = nullptr;
    a.scratch = scr;
    mark(0, st);
    if (n > 0 && (e = launch_msv_exact(a, nwarps_exact, st))) return cuda_status(e);
    mark(1, st);
  }
  return HMG_OK;
}

// sequences the fast kernel flagged (every cell <= B') are rescored exactly (rare)
hmg_status run_msv_redo(const hmg_profile* p, const hmg_db* db, cudaStream_t st, uint8_t* raw_sorted, Scratch& S) {
  cudaError_t e = cudaSuccess;
  const int64_t n = db->nseq;
  if (msv_fast_on(p, db)) {
    MsvArgs a = msv_args(p, db);
    a.raw = raw_sorted;
    const int nwarps_exact = 148 * 16;
    auto* list = (int32_t*)S.get(sizeof(int32_t) * (size_t)std::max<int64_t>(n, 1), &e);
    auto* cnt = (int64_t*)S.get(sizeof(int64_t), &e);
    void* tmp = S.get(scan_tmp_bytes(n) + (size_t)n + 16, &e);
    auto* scr = (uint8_t*)S.get((size_t)nwarps_exact * 2 * (p->M + 1), &e);
    if (e) return cuda_status(e);
    if ((e = select_redo(raw_sorted, n, list, cnt, tmp, st))) return cuda_status(e);
    a.list = list;
    a.nlist = cnt;
    a.scratch = scr;
    if ((e = launch_msv_exact(a, nwarps_exact, st))) return cuda_status(e);
  }
  mark(2, st);
  return HMG_OK;
}

hmg_status run_msv_long_chunks(const hmg_profile* p, const hmg_db* db, cudaStream_t st, uint8_t* raw_sorted,
                               Scratch& S, LongArgs* la_out);

// MSV over the whole DB: the longest sequences as parallel row chunks (long.cu), the rest with
// the lane-group kernel; then the exact re-score of flagged sequences.
hmg_status run_msv(const hmg_profile* p, const hmg_db* db, cudaStream_t st, uint8_t* raw_sorted, Scratch& S) {
  int64_t nlong = -1;
  mark(0, st);
  if (p->long_QV > 0 && msv_fast_on(p, db) && db->nlong > 0 && !tune_int("NO_LONG_LANE", 0)) {
    LongArgs la{};
    hmg_status s = run_msv_long_chunks(p, db, st, raw_sorted, S, &la);
    if (s != HMG_OK) return s;
    nlong = db->nlong;
  }
  hmg_status s = run_msv_fast(p, db, st, raw_sorted, S, nlong, false, false);
  if (s != HMG_OK) return s;
  return run_msv_redo(p, db, st, raw_sorted, S);
}

// set up the long-lane arguments (scratch on S) and launch the chunked MSV on st
hmg_status run_msv_long_chunks(const hmg_profile* p, const hmg_db* db, cudaStream_t st, uint8_t* raw_sorted,
                               Scratch& S, LongArgs* la_out) {
  cudaError_t e = cudaSuccess;
  const int64_t nlong = db->nlong;
  auto* owned = (uint8_t*)S.get((size_t)nlong, &e);
  auto* lctr = (unsigned long long*)S.get(sizeof(unsigned long long) * 2, &e);
  auto* cmax = (int*)S.get(sizeof(int) * (size_t)std::max<int64_t>(db->nchunks, 1), &e);
  auto* cdone = (unsigned*)S.get(sizeof(unsigned) * (size_t)nlong, &e);
  if (e) return cuda_status(e);
  if ((e = cudaMemsetAsync(lctr, 0, sizeof(unsigned long long) * 2, st))) return cuda_status(e);
  if ((e = cudaMemsetAsync(cdone, 0, sizeof(unsigned) * (size_t)nlong, st))) return cuda_status(e);
  LongArgs& la = *la_out;
  la = LongArgs{};
  la.m = msv_args(p, db);
  la.m.prof = p->d_long_msv;
  la.m.raw = raw_sorted;
  la.owned = owned;
  la.nlong = nlong;
  la.chunk_start = db->d_chunk_start;
  la.nitems = db->nchunks;
  la.chunk_rows = db->chunk_rows;
  la.chunk_max = cmax;
  la.chunk_done = cdone;
  la.counter = lctr;
  int ok = 0;
  if ((e = launch_pipe_long_msv(p->long_QL, la, st, &ok))) return cuda_status(e);
  return ok ? HMG_OK : HMG_EUNSUPPORTED;
}

// s32 Viterbi kernels (register / block / generic) for the profile's geometry
hmg_status launch_vit_s32(const hmg_profile* p, VitArgs a, cudaStream_t st, Scratch& S) {
  cudaError_t e = cudaSuccess;
  a.rsc = p->d_rsc;
  a.tr = p->d_tr;
  auto* ctr = (unsigned long long*)S.get(sizeof(unsigned long long), &e);
  if (e) return cuda_status(e);
  if ((e = cudaMemsetAsync(ctr, 0, sizeof(unsigned long long), st))) return cuda_status(e);
  a.counter = ctr;
  if (!p->vit_generic && p->vit_W > 0) {
    int ok = 0;
    if ((e = launch_vit_cta(p->vit_W, p->vit_Q, a, st, &ok))) return cuda_status(e);
    if (!ok) return HMG_EUNSUPPORTED;
  } else if (!p->vit_generic) {
    int ok = 0;
    if ((e = launch_vit_reg(p->vit_G, p->vit_Q, a, st, &ok))) return cuda_status(e);
    if (!ok) return HMG_EUNSUPPORTED;
  } else {
    const int nwarps = 148 * 16;
    auto* scr = (int32_t*)S.get((size_t)nwarps * 6 * (p->M + 1) * sizeof(int32_t), &e);
    if (e) return cuda_status(e);
    a.scratch = scr;
    if ((e = launch_vit_generic(a, nwarps, st))) return cuda_status(e);
  }
  return HMG_OK;
}

// Viterbi over sorted-order ids (list, device count) into raw_sorted.  With the s16x2 pair kernel
// the sequences it cannot score exactly in its 16-bit window (vit_pair.cuh) are re-scored by the
// s32 kernel from a device list (launched unconditionally; it exits at once when the list is empty).
hmg_status run_vit(const hmg_profile* p, const hmg_db* db, const int32_t* list, const int64_t* nlist,
                   cudaStream_t st, int16_t* raw_sorted, Scratch& S, const uint8_t* done = nullptr,
                   int64_t ndone = 0, bool marks = true, int64_t cap = -1) {
  cudaError_t e = cudaSuccess;
  VitArgs a{};
  a.words = db->d_words;
  a.woff16 = db->d_woff16;
  a.len = db->d_len;
  a.nseq = db->nseq;
  a.move = db->d_move;
  a.M = p->M;
  a.list = list;
  a.nlist = nlist;
  a.raw_sorted = raw_sorted;
  a.done = done;
  a.ndone = done ? ndone : 0;
  if (marks) mark(3, st);
  hmg_status s = HMG_OK;
  if (p->pair_G > 0) {
    if (cap < 0) cap = db->nseq;                      // redo list capacity: entries of the id list
    auto* ctr = (unsigned long long*)S.get(sizeof(unsigned long long) * 2, &e);
    auto* redo = (int32_t*)S.get(sizeof(int32_t) * (size_t)std::max<int64_t>(cap, 1), &e);
    if (e) return cuda_status(e);
    if ((e = cudaMemsetAsync(ctr, 0, sizeof(unsigned long long) * 2, st))) return cuda_status(e);
    VitArgs b = a;
    b.rsc = reinterpret_cast<const int16_t*>(p->d_pair_rsc);
    b.tr = reinterpret_cast<const int32_t*>(p->d_pair_tr);
    b.counter = ctr;
    b.tbm_min = p->tbm_min;
    b.safe = 32767 - p->rmax;
    b.redo_list = redo;
    b.redo_count = ctr + 1;
    int ok = 0;
    if (p->pair_wide) {
      if ((e = launch_vit_wide(p->pair_Q, p->pair_wide == 2, b, st, &ok))) return cuda_status(e);
    } else if (p->pair_SG2 > 0) {
      if ((e = launch_vit_cpair2(p->pair_SG2, p->pair_Q, b, st, &ok))) return cuda_status(e);
    } else if (p->pair_W > 0) {
      if ((e = launch_vit_cpair(p->pair_W, p->pair_SG, p->pair_Q, b, st, &ok))) return cuda_status(e);
    } else {
      if ((e = launch_vit_pair(p->pair_G, p->pair_Q, p->pair_scan, b, st, &ok))) return cuda_status(e);
    }
    if (!ok) return HMG_EUNSUPPORTED;
    stage_count_redo(ctr + 1, st);
    VitArgs r = a;                                   // re-score list: never in the long lane
    r.list = redo;
    r.nlist = reinterpret_cast<const int64_t*>(ctr + 1);
    r.done = nullptr;
    r.ndone = 0;
    s = launch_vit_s32(p, r, st, S);
  } else {
    s = launch_vit_s32(p, a, st, S);
  }
  if (s != HMG_OK) return s;
  if (marks) mark(4, st);
  return HMG_OK;
}

bool bad_float(float v, bool allow_pos) {
  if (std::isnan(v)) return true;
  if (v == INFINITY) return true;
  if (!allow_pos && v > 0.0f) return true;
  return false;
}

}  // namespace

// =====================================================================================
extern "C" {

const char* hmg_strerror(hmg_status s) {
  switch (s) {
    case HMG_OK: return "ok";
    case HMG_EINVAL: return "invalid argument";
    case HMG_ENOMEM: return "out of memory";
    case HMG_ECUDA: return "CUDA error";
    case HMG_EUNSUPPORTED: return "unsupported";
  }
  return "unknown status";
}

int64_t hmg_kernel_launches(void) { return g_launches.load(); }

hmg_status hmg_set_tuning(const char* name, int value) {
  if (!name || !tune_known(name)) return HMG_EINVAL;
  std::lock_guard<std::mutex> g(g_tune_mu);
  g_tune[name] = value;
  return HMG_OK;
}

hmg_status hmg_clear_tuning(const char* name) {
  std::lock_guard<std::mutex> g(g_tune_mu);
  if (!name) {
    g_tune.clear();
    return HMG_OK;
  }
  if (!tune_known(name)) return HMG_EINVAL;
  g_tune.erase(name);
  return HMG_OK;
}

hmg_status hmg_prepare_thresholds(const hmg_profile* pc, double F1, double F2, int Lmax) {
  hmg_profile* p = const_cast<hmg_profile*>(pc);
  if (!p || !p->has_ev || p->device < 0 || Lmax < 1 || !(F1 > 0.0 && F1 <= 1.0) || !(F2 > 0.0 && F2 <= 1.0))
    return HMG_EINVAL;
  Dev dg(p->device);
  const uint16_t* tm = nullptr;
  hmg_status s = msv_thr_table(p, nullptr, F1, &tm, nullptr, Lmax);
  if (s == HMG_OK && p->has_tsc) {
    const int32_t* tv = nullptr;
    s = vit_thr_table(p, nullptr, F2, &tv, nullptr, Lmax);
  }
  return s;
}

hmg_status hmg_set_stage_timing(int enable) {
  std::lock_guard<std::mutex> g(g_timer_mu);
  if (enable && !g_timer.on) {
    cudaGetDevice(&g_timer.device);
    for (auto& e : g_timer.ev)
      if (cudaEventCreate(&e) != cudaSuccess) return cuda_status(cudaGetLastError());
    if (cudaMallocHost(&g_timer.h_redo, sizeof(unsigned long long)) != cudaSuccess)
      return cuda_status(cudaGetLastError());
    g_timer.on = true;
  } else if (!enable && g_timer.on) {
    for (auto& e : g_timer.ev) cudaEventDestroy(e);
    cudaFreeHost(g_timer.h_redo);
    g_timer = StageTimer();
  }
  return HMG_OK;
}

hmg_status hmg_stage_times(double* ms) {
  if (!ms) return HMG_EINVAL;
  std::lock_guard<std::mutex> g(g_timer_mu);
  if (!g_timer.on) return HMG_EINVAL;
  for (int i = 0; i < kStages; ++i) ms[i] = -1.0;
  int last = -1;
  for (int i = kStages; i >= 0; --i)
    if (g_timer.rec[i]) { last = i; break; }
  if (last < 0) return HMG_OK;
  if (cudaEventSynchronize(g_timer.ev[last]) != cudaSuccess) return cuda_status(cudaGetLastError());
  for (int i = 0; i < kStages; ++i) {
    if (!g_timer.rec[i] || !g_timer.rec[i + 1]) continue;
    float t = 0.f;
    if (cudaEventElapsedTime(&t, g_timer.ev[i], g_timer.ev[i + 1]) == cudaSuccess) ms[i] = t;
    else cudaGetLastError();
  }
  return HMG_OK;
}

hmg_status hmg_stage_counts(int64_t* counts) {
  if (!counts) return HMG_EINVAL;
  std::lock_guard<std::mutex> g(g_timer_mu);
  if (!g_timer.on) return HMG_EINVAL;
  counts[0] = -1;
  int last = -1;
  for (int i = kStages; i >= 0; --i)
    if (g_timer.rec[i]) { last = i; break; }
  if (last >= 0 && cudaEventSynchronize(g_timer.ev[last]) != cudaSuccess) return cuda_status(cudaGetLastError());
  if (g_timer.redo_rec) counts[0] = (int64_t)*g_timer.h_redo;
  return HMG_OK;
}

float hmg_msv_nats(int raw, int L) { return msv_nats_of(raw, L); }
float hmg_vit_nats(int raw, int L) { return vit_nats_of(raw, L); }
float hmg_null1_nats(int L) { return null1_of(L); }
double hmg_gumbel_surv(double bits, double mu, double lambda) { return gumbel_surv(bits, mu, lambda); }

hmg_status hmg_profile_create(int M, const float* msc, const float* tsc, const hmg_evparams* ev, int device,
                              hmg_profile** out) {
  if (!out || !msc || M < 1 || M > 100000) return HMG_EINVAL;
  *out = nullptr;
  for (size_t i = 0; i < (size_t)M * kAlpha; ++i)
    if (bad_float(msc[i], true)) return HMG_EINVAL;
  if (tsc)
    for (size_t i = 0; i < (size_t)M * 8; ++i)
      if (bad_float(tsc[i], false)) return HMG_EINVAL;
  if (ev && (!(ev->lambda_msv > 0) || !(ev->lambda_vit > 0) || std::isnan(ev->mu_msv) || std::isnan(ev->mu_vit)))
    return HMG_EINVAL;
  if (device >= 0) {   // device < 0: host-only handle (quantised tables, no device copies)
    int ndev = 0;
    if (cudaGetDeviceCount(&ndev) != cudaSuccess || device >= ndev) {
      cudaGetLastError();
      return ndev == 0 ? HMG_EUNSUPPORTED : HMG_EINVAL;
    }
  }
  if (device >= 0) keep_pool_cached(device);
  hmg_profile* p = new (std::nothrow) hmg_profile();
  if (!p) return HMG_ENOMEM;
  p->M = M;
  p->device = device;
  const Scales S;
  p->scale_b = S.b;
  p->scale_w = S.w;
  // ---- byte profile (R1, R3, R4, R7)
  float best = 0.0f;
  for (int k = 0; k < M; ++k)
    for (int x = 0; x < 20; ++x) best = std::max(best, msc[(size_t)k * kAlpha + x]);
  p->bias = cost_unbiased(-best, S);
  p->tbm = cost_unbiased(logf(2.0f / ((float)M * (float)(M + 1))), S);
  p->tec = cost_unbiased(logf(0.5f), S);
  p->cost.resize((size_t)kAlpha * M);
  for (int x = 0; x < kAlpha; ++x)
    for (int k = 0; k < M; ++k) p->cost[(size_t)x * M + k] = cost_biased(msc[(size_t)k * kAlpha + x], p->bias, S);
  // ---- word profile (R2, R5, R6)
  p->rsc.resize((size_t)kAlpha * M);
  for (int x = 0; x < kAlpha; ++x)
    for (int k = 0; k < M; ++k) p->rsc[(size_t)x * M + k] = word(msc[(size_t)k * kAlpha + x], S);
  p->has_tsc = tsc != nullptr;
  if (tsc) {
    p->tsc.resize((size_t)8 * M);
    for (int t = 0; t < 8; ++t)
      for (int k = 0; k < M; ++k) {
        int v = word(tsc[(size_t)k * 8 + t], S);
        const int cap = t == 6 ? -1 : (t == 7 ? 32767 : 0);
        p->tsc[(size_t)t * M + k] = (int16_t)std::min(v, cap);
      }
    int ddb = -32768;
    for (int k = 2; k <= M - 2; ++k) {
      const int v = (int)word(tsc[(size_t)(k - 1) * 8 + 7], S) + (int)word(tsc[(size_t)(k + 1) * 8 + 3], S) -
                    (int)word(tsc[(size_t)(k + 1) * 8 + 0], S);
      ddb = std::max(ddb, v);
    }
    p->ddbound = ddb;
  }
  if (ev) {
    p->has_ev = true;
    p->ev = *ev;
  }
  p->msc_max = -INFINITY;
  for (size_t i = 0; i < (size_t)M * kAlpha; ++i) p->msc_max = std::max(p->msc_max, msc[i]);
  // ---- Forward stage geometry (forward.cu): emission rows staged in shared memory as fit
  const int fwd_qmax = tune_int("FWD_QMAX", 16) >= 16 ? 16 : 8;   // 16: profiles/fwd_bench_r01e.jsonl
  if (tsc && (fwd_geometry(M, &p->fwd_T, &p->fwd_Q, fwd_qmax) || fwd_geometry(M, &p->fwd_T, &p->fwd_Q, 8))) {
    const int wo = tune_int("FWD_W", 0);   // whole warps per sequence (1 = no sub-warp groups)
    if (wo == 1 || wo == 2 || wo == 4 || wo == 8 || wo == 16) {
      int q = 2;
      while (32 * wo * q < M && q < 16) q *= 2;
      if (32 * wo * q >= M) {
        p->fwd_T = 32 * wo;
        p->fwd_Q = q;
      }
    }
    int smax = 0;
    if (device >= 0) cudaDeviceGetAttribute(&smax, cudaDevAttrMaxSharedMemoryPerBlockOptin, device);
    else smax = 227 * 1024;
    int rows = kAlpha;
    while (rows > 0 && fwd_smem(p->fwd_T, p->fwd_Q, rows, 1) > (size_t)smax) --rows;
    p->fwd_rows = rows;
    p->fwd_W = p->fwd_T >= 32 ? p->fwd_T / 32 : 1;
    if (device >= 0) {
      Dev dg(device);
      p->fwd_S = fwd_pick_s(p->fwd_T, p->fwd_Q, rows);
      const int so = tune_int("FWD_S", 0);
      if (so > 0) p->fwd_S = so;
      if (p->fwd_S == 0) p->fwd_W = p->fwd_T = 0;   // no launchable configuration: Forward unsupported
    }
  }
  // ---- kernel geometry and device tables
  p->msv_fast = p->bias < 66 + p->tbm;   // precondition of the fast MSV kernel
  msv_geometry(M, &p->msv_G, &p->msv_Q);
  if (tsc) {
    vit_geometry(M, &p->vit_G, &p->vit_Q);
    if (p->vit_Q == 0 || tune_int("VIT_CTA", 0)) {   // long models: block-per-sequence kernel
      int W = M <= 2048 ? 8 : 16;           // W = 8 keeps two 256-thread blocks per SM up to M = 2048
      const int wo = tune_int("VIT_CTA_W", 0);
      if (wo == 4 || wo == 8 || wo == 16) W = wo;
      int Q = (M + 32 * W - 1) / (32 * W);
      Q += Q & 1;
      int smax = 0;   // the s16 emission table must fit in one block's shared memory
      if (device >= 0) cudaDeviceGetAttribute(&smax, cudaDevAttrMaxSharedMemoryPerBlockOptin, device);
      else smax = 227 * 1024;
      if (Q <= 8 && vit_cta_smem(W, Q) <= (size_t)smax) {
        p->vit_W = W;
        p->vit_G = 32 * W;
        p->vit_Q = Q;
      } else {
        p->vit_Q = 0;
      }
    }
    p->vit_generic = p->vit_Q == 0 || tune_int("VIT_GENERIC", 0);
    // s16x2 pair kernel (vit_pair.cuh) in front of the s32 kernels: its 16-bit window must hold
    // xN + move(L) + tBM_k .. 32767 for typical L, so entry scores and emissions must be moderate
    int tmin = 32767, rmx = 0;
    for (int k = 0; k < M; ++k) tmin = std::min(tmin, (int)p->tsc[k]);
    for (int16_t v : p->rsc) rmx = std::max(rmx, (int)v);
    p->tbm_min = tmin;
    p->rmax = rmx;
    if (tmin > -16384 && rmx < 8192 && !tune_int("NO_VIT_PAIR", 0)) {
      // lane-group size from the sweep (profiles/vit_pair_sweep_r01.jsonl): registers per lane
      // (12 Q + ~30) set the warps per SM, so small Q (4-8) wins over fewer lanes per sequence
      int g = M <= 64 ? 8 : M <= 128 ? 16 : 32;
      const int o = tune_int("VIT_PAIR_G", 0);
      if (o == 8 || o == 16 || o == 32) g = o;
      int q = (M + 2 * g - 1) / (2 * g);
      while (q > vit_pair_q_max() && g < 32) {
        g *= 2;
        q = (M + 2 * g - 1) / (2 * g);
      }
      if (q <= vit_pair_q_max() && !tune_int("VIT_PAIR_CTA", 0)) {
        p->pair_G = g;
        p->pair_Q = q;
        // Lazy-F by max-plus scan (f1) when D->D chains are long: its cost does not depend on the
        // profile, the vote-terminated passes win on typical ones (profiles/vit_scan_f1_r01.jsonl)
        double pdd = 0.0;
        for (int k = 0; k + 1 < M; ++k) pdd += std::exp((double)tsc[(size_t)k * 8 + 7]);
        pdd = M > 1 ? pdd / (M - 1) : 0.0;
        p->pair_scan = g == 32 && tune_int("VIT_SCAN", pdd > 0.6 ? 1 : 0);
      } else {   // long models: block-per-sequence pair kernel, W warps on one DP row
        // W warps per sequence and SG sequences per block from the sweep on the config-4 shape
        // (profiles/vit_cpair_sweep_r01.jsonl): 2 warps x 16 registers per thread, 2 sequences
        // per block sharing the table, up to M = 2048; wider rows above
        int W = M <= 2048 ? 2 : 4, SG = M <= 2048 ? 2 : 1;
        const int wo = tune_int("VIT_PAIR_W", 0);
        if (wo == 2 || wo == 4 || wo == 8 || wo == 16) {
          W = wo;
          SG = W == 2 ? 2 : W == 4 ? 3 : W == 8 ? 2 : 1;
        }
        SG = tune_int("VIT_PAIR_SG", SG);
        int qq = std::max(2, (M + 64 * W - 1) / (64 * W));
        while (!vit_cpair_available(W, SG, qq) && W < 16) {   // models too long for W warps
          W *= 2;
          SG = 1;
          qq = std::max(2, (M + 64 * W - 1) / (64 * W));
        }
        int smax = 0;
        if (device >= 0) cudaDeviceGetAttribute(&smax, cudaDevAttrMaxSharedMemoryPerBlockOptin, device);
        else smax = 227 * 1024;
        if (vit_cpair_available(W, SG, qq) && vit_cpair_smem(W, SG, qq) <= (size_t)smax) {
          p->pair_W = W;
          p->pair_SG = SG;
          p->pair_G = 32 * W;
          p->pair_Q = qq;
        }
        // two warps: the kernel without a per-row barrier (vit_cpair2.cuh) unless asked otherwise
        const int sg2 = tune_int("VIT_CPAIR2", 2);
        if (p->pair_W == 2 && sg2 > 0 && vit_cpair2_available(sg2, qq) && vit_cpair2_smem(sg2, qq) <= (size_t)smax)
          p->pair_SG2 = sg2;
        // one warp per sequence, transitions in tensor (VIT_WIDE = 2) or shared memory (1)
        // (vit_wide.cuh): 64 Q4 >= M.  Default from profiles/wide_r02zc.jsonl (100k sequences):
        // M = 2048 TMEM 2 775 GCUPS vs shared 2 233 vs two warps 2 204; M = 1500 2 622 / 2 268 /
        // 1 847; M = 1100 (Q4 = 20) 2 227 / 2 318 / 1 839
        const int q4 = ((M + 63) / 64 + 3) / 4 * 4;
        const int wide = tune_int("VIT_WIDE", q4 >= 24 ? 2 : 1);
        if ((wide == 1 || wide == 2) && vit_wide_available(q4) && vit_wide_smem(q4, wide == 2) <= (size_t)smax) {
          p->pair_wide = wide;
          p->pair_W = 0;
          p->pair_SG2 = 0;
          p->pair_G = 32;
          p->pair_Q = q4;
        }
      }
    }
  }
  if (device < 0) {
    *out = p;
    return HMG_OK;
  }
  Dev dg(device);
  hmg_status st = HMG_OK;
  {
    std::vector<uint8_t> c((size_t)kRows * M, 255);
    std::copy(p->cost.begin(), p->cost.end(), c.begin());
    st = upload(&p->d_cost, c.data(), c.size());
  }
  if (st == HMG_OK && p->msv_Q > 0) {
    auto t = msv_table(*p, p->msv_G, p->msv_Q);
    if (p->msv_G < 32) {   // second table for the whole-warp (G = 32) long-sequence queue
      const int QL = (p->msv_G * p->msv_Q + 31) / 32;
      auto t2 = msv_table(*p, 32, QL);
      t.insert(t.end(), t2.begin(), t2.end());
    }
    p->msv_prof_bytes = t.size() * 4;
    st = upload(&p->d_msv_prof, t.data(), t.size());
  }
  if (st == HMG_OK && tsc) {
    if (!p->vit_generic && p->vit_W > 0) {
      std::vector<uint32_t> r;
      std::vector<int32_t> t;
      vit_tables_s16(*p, p->vit_G, p->vit_Q, &r, &t);
      p->vit_rsc_bytes = r.size() * 4;
      p->vit_tr_bytes = t.size() * 4;
      st = upload(reinterpret_cast<uint32_t**>(&p->d_rsc), r.data(), r.size());
      if (st == HMG_OK) st = upload(&p->d_tr, t.data(), t.size());
    } else if (!p->vit_generic) {
      std::vector<uint32_t> r;
      std::vector<int32_t> t;
      vit_tables(*p, p->vit_G, p->vit_Q, &r, &t);
      p->vit_rsc_bytes = r.size() * 4;
      p->vit_tr_bytes = t.size() * 4;
      st = upload(reinterpret_cast<uint32_t**>(&p->d_rsc), r.data(), r.size());
      if (st == HMG_OK) st = upload(&p->d_tr, t.data(), t.size());
    } else {
      std::vector<int16_t> r((size_t)kRows * M, (int16_t)kNegW);
      std::copy(p->rsc.begin(), p->rsc.end(), r.begin());
      std::vector<int32_t> t(p->tsc.begin(), p->tsc.end());
      st = upload(&p->d_rsc, r.data(), r.size());
      if (st == HMG_OK) st = upload(&p->d_tr, t.data(), t.size());
    }
  }
  if (st == HMG_OK && tsc && p->pair_G > 0) {
    std::vector<uint32_t> r, t;
    vit_pair_tables(*p, p->pair_G, p->pair_Q, &r, &t);
    st = upload(&p->d_pair_rsc, r.data(), r.size());
    if (st == HMG_OK) st = upload(&p->d_pair_tr, t.data(), t.size());
  }
  // pipeline long lane: whole-warp Viterbi with the pair lane (the pair tables when G = 32, models
  // up to 1024 nodes) or the s32 latency lane (models up to 512 nodes)
  const bool lpair = p->pair_G == 32 && p->pair_W == 0 && !p->pair_wide && !tune_int("LONG_S32", 0);
  // models whose pair kernel uses lane groups (M <= 128): the long lane gets pair tables of its own
  // in the whole-warp geometry (G = 32, ceil(M / 64) registers)
  const bool lpair_own = !lpair && p->pair_G > 0 && p->pair_G < 32 && !tune_int("LONG_S32", 0) &&
                         tune_int("LONG_PAIR_SMALL", 1);
  if (st == HMG_OK && tsc && (lpair || M <= 512) && !tune_int("NO_LONG_LANE", 0)) {
    const int QL = long_msv_q(M);
    auto tm = msv_table(*p, 32, QL);
    st = upload(&p->d_long_msv, tm.data(), tm.size());
    if (lpair) {
      if (st == HMG_OK) {
        p->long_QV = p->pair_Q;
        p->long_pair = true;
        p->long_QL = QL;
      }
    } else if (lpair_own) {
      const int Q32 = (M + 63) / 64;
      std::vector<uint32_t> r, t;
      vit_pair_tables(*p, 32, Q32, &r, &t);
      if (st == HMG_OK) st = upload(reinterpret_cast<uint32_t**>(&p->d_long_rsc), r.data(), r.size());
      if (st == HMG_OK) st = upload(reinterpret_cast<uint32_t**>(&p->d_long_tr), t.data(), t.size());
      if (st == HMG_OK) {
        p->long_QV = Q32;
        p->long_pair = true;
        p->long_QL = QL;
      }
    } else {
      const int QV = (M + 31) / 32;
      std::vector<uint32_t> r;
      std::vector<int32_t> t;
      vit_tables(*p, 32, QV, &r, &t);
      if (st == HMG_OK) st = upload(reinterpret_cast<uint32_t**>(&p->d_long_rsc), r.data(), r.size());
      if (st == HMG_OK) st = upload(&p->d_long_tr, t.data(), t.size());
      if (st == HMG_OK) {
        p->long_QV = QV;
        p->long_QL = QL;
      }
    }
  }
  if (st == HMG_OK && p->fwd_W > 0) {
    std::vector<float> e, t, c;
    fwd_tables(M, p->fwd_T, p->fwd_Q, msc, tsc, &e, &t, &c);
    st = upload(&p->d_fwd_e, e.data(), e.size());
    if (st == HMG_OK) st = upload(&p->d_fwd_t, t.data(), t.size());
    if (st == HMG_OK) st = upload(&p->d_fwd_c, c.data(), c.size());
  }
  if (st != HMG_OK) {
    hmg_profile_destroy(p);
    return st;
  }
  *out = p;
  return HMG_OK;
}

hmg_status hmg_calibrate_db(const hmg_profile* p, const hmg_db* db, double lambda, hmg_evparams* out) {
  if (!p || !db || !out || !(lambda > 0) || !p->has_tsc || p->device < 0 || db->device != p->device ||
      db->nseq < 1)
    return HMG_EINVAL;
  const int64_t n = db->nseq;
  Dev dg(p->device);
  uint8_t* d_m = nullptr;
  int16_t* d_v = nullptr;
  hmg_status s = HMG_OK;
  cudaError_t e = cudaMalloc(&d_m, (size_t)n);
  if (e == cudaSuccess) e = cudaMalloc(&d_v, sizeof(int16_t) * (size_t)n);
  if (e == cudaSuccess) {
    s = hmg_msv(p, db, 0.02, nullptr, d_m, nullptr);
    if (s == HMG_OK) s = hmg_viterbi(p, db, nullptr, 0, 1e-3, nullptr, d_v, nullptr);
  } else {
    s = cuda_status(e);
  }
  std::vector<uint8_t> hm((size_t)n);
  std::vector<int16_t> hv((size_t)n);
  if (s == HMG_OK) {
    e = cudaMemcpy(hm.data(), d_m, (size_t)n, cudaMemcpyDeviceToHost);
    if (e == cudaSuccess) e = cudaMemcpy(hv.data(), d_v, sizeof(int16_t) * (size_t)n, cudaMemcpyDeviceToHost);
    s = cuda_status(e);
  }
  cudaFree(d_m);
  cudaFree(d_v);
  if (s != HMG_OK) return s;
  std::vector<int> len((size_t)n);                 // caller-order lengths
  for (int64_t j = 0; j < n; ++j) len[(size_t)db->order[(size_t)j]] = db->len_sorted[(size_t)j];
  // closed-form ML location of a Gumbel with known lambda over the finite bit scores
  auto fit = [&](auto nats_of, const auto& raw) {
    double acc = 0;
    int64_t cnt = 0;
    for (int64_t j = 0; j < n; ++j) {
      const int L = len[(size_t)j];
      const float nats = nats_of((int)raw[(size_t)j], L);
      if (!std::isfinite(nats)) continue;
      acc += exp(-lambda * ((double)(nats - null1_of(L)) / kLn2));
      ++cnt;
    }
    return cnt ? -log(acc / (double)cnt) / lambda : 0.0;
  };
  out->mu_msv = fit(msv_nats_of, hm);
  out->mu_vit = fit(vit_nats_of, hv);
  out->lambda_msv = out->lambda_vit = lambda;
  return HMG_OK;
}

hmg_status hmg_calibrate(const hmg_profile* p, int n, int L, uint64_t seed, double lambda, hmg_evparams* out) {
  if (!p || !out || n < 1 || L < 1 || !(lambda > 0) || !p->has_tsc || p->device < 0) return HMG_EINVAL;
  // HMMER3 amino background (reading R34) and 0.05% X, as the synthetic databases
  static const double f[20] = {0.0787945, 0.0151600, 0.0535222, 0.0668298, 0.0397062, 0.0695071, 0.0229198,
                               0.0590092, 0.0594422, 0.0963728, 0.0237718, 0.0414386, 0.0482904, 0.0395639,
                               0.0540978, 0.0683364, 0.0540687, 0.0673417, 0.0114135, 0.0304133};
  std::vector<double> w(f, f + 20);
  double tot = 0;
  for (double v : w) tot += v;
  for (double& v : w) v = v / tot * (1.0 - 0.0005);
  w.push_back(0.0005);
  std::mt19937_64 rng(seed);
  std::discrete_distribution<int> pick(w.begin(), w.end());
  std::vector<uint8_t> dsq((size_t)n * L);
  for (auto& c : dsq) {
    const int k = pick(rng);
    c = (uint8_t)(k == 20 ? 26 : k);
  }
  std::vector<int64_t> off((size_t)n + 1);
  for (int i = 0; i <= n; ++i) off[i] = (int64_t)i * L;
  hmg_db* db = nullptr;
  hmg_status s = hmg_db_create(dsq.data(), off.data(), n, p->device, &db);
  if (s != HMG_OK) return s;
  s = hmg_calibrate_db(p, db, lambda, out);
  hmg_db_destroy(db);
  return s;
}

hmg_status hmg_profile_quant(const hmg_profile* p, hmg_quant* q) {
  if (!p || !q) return HMG_EINVAL;
  q->M = p->M;
  q->bias_b = p->bias;
  q->tbm_b = p->tbm;
  q->tec_b = p->tec;
  q->base_b = kBaseB;
  q->scale_b = p->scale_b;
  q->base_w = kBaseW;
  q->xw_e = word(logf(0.5f), Scales());
  q->ddbound_w = p->ddbound;
  q->scale_w = p->scale_w;
  q->cost = p->cost.data();
  q->rsc = p->rsc.data();
  q->tsc = p->has_tsc ? p->tsc.data() : nullptr;
  q->msv_fast = p->msv_fast;
  q->msv_lanes = p->msv_G;
  q->msv_regs = p->msv_Q;
  q->vit_lanes = p->vit_generic ? 32 : p->vit_G;   // block kernel: 32 * warps
  q->vit_nodes = p->vit_generic ? 0 : p->vit_Q;
  q->vit_pair_lanes = p->pair_G;
  q->vit_pair_regs = p->pair_Q;
  q->vit_pair_kernel = p->pair_G == 0 ? 0
                       : p->pair_wide ? 3 + p->pair_wide
                       : p->pair_SG2 > 0 ? 3
                       : p->pair_W > 0 ? 2 : 1;
  q->fwd_warps = p->fwd_W;
  q->fwd_lanes = p->fwd_T;
  q->fwd_nodes = p->fwd_Q;
  q->fwd_rows_smem = p->fwd_rows;
  q->fwd_seqs_per_block = p->fwd_S;
  return HMG_OK;
}

void hmg_profile_destroy(hmg_profile* p) {
  if (!p) return;
  if (p->device >= 0) {
    Dev dg(p->device);
    cudaFree(p->d_msv_prof);
    cudaFree(p->d_cost);
    cudaFree(p->d_rsc);
    cudaFree(p->d_tr);
    cudaFree(p->d_long_msv);
    cudaFree(p->d_long_rsc);
    cudaFree(p->d_long_tr);
    cudaFree(p->d_pair_rsc);
    cudaFree(p->d_pair_tr);
    cudaFree(p->d_fwd_e);
    cudaFree(p->d_fwd_t);
    cudaFree(p->d_fwd_c);
    for (auto& t : p->msv_tabs) cudaFree(t.d);
    for (auto& t : p->thr_msv) cudaFree(t.d);
    for (auto& t : p->thr_vit) cudaFree(t.d);
    cudaGetLastError();
  }
  delete p;
}

hmg_status hmg_db_create(const uint8_t* dsq, const int64_t* off, int64_t nseq, int device, hmg_db** out) {
  if (!out || nseq < 0 || (nseq > 0 && (!dsq || !off)) || nseq > 0x7fffffff) return HMG_EINVAL;
  *out = nullptr;
  if (device >= 0) {   // device < 0: host-only handle (packed image kept on the host)
    int ndev = 0;
    if (cudaGetDeviceCount(&ndev) != cudaSuccess || device >= ndev) {
      cudaGetLastError();
      return ndev == 0 ? HMG_EUNSUPPORTED : HMG_EINVAL;
    }
  }
  // validate (codes 0..28; lengths >= 1)
  int64_t res = 0;
  int Lmax = 0;
  for (int64_t s = 0; s < nseq; ++s) {
    const int64_t L = off[s + 1] - off[s];
    if (L < 1 || L > 0x3fffffff || off[s] < 0) return HMG_EINVAL;
    Lmax = std::max<int64_t>(Lmax, L);
    res += L;
  }
  for (int64_t i = 0; i < (nseq ? off[nseq] - off[0] : 0); ++i)
    if (dsq[off[0] + i] > 28) return HMG_EINVAL;
  if (device >= 0) keep_pool_cached(device);
  hmg_db* db = new (std::nothrow) hmg_db();
  if (!db) return HMG_ENOMEM;
  db->device = device;
  db->nseq = nseq;
  db->residues = res;
  db->Lmax = Lmax;
  // length sort, descending, stable (schedule order)
  db->order.resize(nseq);
  std::iota(db->order.begin(), db->order.end(), 0);
  std::stable_sort(db->order.begin(), db->order.end(), [&](int32_t a, int32_t b) {
    return off[a + 1] - off[a] > off[b + 1] - off[b];
  });
  db->len_sorted.resize(nseq);
  std::vector<uint32_t> woff16(nseq);
  int64_t words = 0;
  for (int64_t j = 0; j < nseq; ++j) {
    const int32_t s = db->order[j];
    const int L = (int)(off[s + 1] - off[s]);
    db->len_sorted[j] = L;
    if (words / 4 > 0xffffffffLL) {
      delete db;
      return HMG_EUNSUPPORTED;
    }
    woff16[j] = (uint32_t)(words / 4);
    words += ((L + 5) / 6 + 3) / 4 * 4;   // 16-byte aligned runs
  }
  db->nwords = words;
  db->woff16_h = woff16;
  // pack 6 residues per word, residue j in bits [5j, 5j+5), pad 31 (Fig 6)
  std::vector<uint32_t> img((size_t)std::max<int64_t>(words, 4), 0xffffffffu);
  for (int64_t j = 0; j < nseq; ++j) {
    const int32_t s = db->order[j];
    const uint8_t* d = dsq + off[s];
    const int L = db->len_sorted[j];
    uint32_t* w = img.data() + (size_t)woff16[j] * 4;
    const int nw = (L + 5) / 6;
    for (int i = 0; i < nw; ++i) {
      uint32_t v = 0;
      for (int b = 0; b < 6; ++b) {
        const int r = 6 * i + b;
        v |= (uint32_t)(r < L ? d[r] : kPadCode) << (5 * b);
      }
      w[i] = v & 0x3fffffffu;
    }
  }
  std::vector<uint8_t> tjb((size_t)Lmax + 1, 0);
  std::vector<int16_t> mv((size_t)Lmax + 1, 0);
  for (int L = 1; L <= Lmax; ++L) {
    tjb[L] = (uint8_t)tjb_of(L);
    mv[L] = move_of(L);
  }
  std::vector<int32_t> inv(nseq);
  for (int64_t j = 0; j < nseq; ++j) inv[db->order[j]] = (int32_t)j;
  // pipeline long lane: L > max(1500, 8 x mean) (env HMG_PIPE_LLONG), chunks of 1032 rows
  std::vector<int32_t> cstart(1, 0);
  {
    const double mean = nseq ? (double)res / (double)nseq : 0.0;
    db->long_cut = tune_int("PIPE_LLONG", (int)std::max(1500.0, 8.0 * mean));
    db->chunk_rows = std::max(6, tune_int("PIPE_CHUNK", 1032) / 6 * 6);
    while (db->nlong < nseq && db->len_sorted[db->nlong] > db->long_cut) {
      const int L = db->len_sorted[db->nlong];
      cstart.push_back(cstart.back() + (L + db->chunk_rows - 1) / db->chunk_rows);
      ++db->nlong;
    }
    db->nchunks = cstart.back();
  }
  if (device < 0) {
    db->host_image = std::move(img);
    *out = db;
    return HMG_OK;
  }
  Dev dg(device);
  hmg_status st = upload(&db->d_words, img.data(), img.size());
  if (st == HMG_OK) st = upload(&db->d_woff16, woff16.data(), woff16.size());
  if (st == HMG_OK) st = upload(&db->d_len, db->len_sorted.data(), db->len_sorted.size());
  if (st == HMG_OK) st = upload(&db->d_order, db->order.data(), db->order.size());
  if (st == HMG_OK) st = upload(&db->d_inv, inv.data(), inv.size());
  if (st == HMG_OK) st = upload(&db->d_tjb, tjb.data(), tjb.size());
  if (st == HMG_OK) st = upload(&db->d_move, mv.data(), mv.size());
  if (st == HMG_OK) st = upload(&db->d_chunk_start, cstart.data(), cstart.size());
  if (st != HMG_OK) {
    hmg_db_destroy(db);
    return st;
  }
  *out = db;
  return HMG_OK;
}

int64_t hmg_db_nseq(const hmg_db* db) { return db ? db->nseq : -1; }
int64_t hmg_db_residues(const hmg_db* db) { return db ? db->residues : -1; }
int64_t hmg_db_packed_bytes(const hmg_db* db) { return db ? std::max<int64_t>(db->nwords, 4) * 4 : -1; }

int64_t hmg_db_long_lane(const hmg_db* db, int64_t* residues) {
  if (!db) return -1;
  if (residues) {
    int64_t r = 0;
    for (int64_t j = 0; j < db->nlong; ++j) r += db->len_sorted[j];
    *residues = r;
  }
  return db->nlong;
}

hmg_status hmg_db_order(const hmg_db* db, int32_t* order) {
  if (!db || (!order && db->nseq)) return HMG_EINVAL;
  std::copy(db->order.begin(), db->order.end(), order);
  return HMG_OK;
}

hmg_status hmg_db_image(const hmg_db* db, uint32_t* image) {
  if (!db || !image) return HMG_EINVAL;
  if (db->device < 0) {
    std::copy(db->host_image.begin(), db->host_image.end(), image);
    return HMG_OK;
  }
  Dev dg(db->device);
  return cuda_status(cudaMemcpy(image, db->d_words, (size_t)hmg_db_packed_bytes(db), cudaMemcpyDeviceToHost));
}

hmg_status hmg_db_upload(hmg_db* db, const uint32_t* image, void* stream) {
  if (!db || !image || db->device < 0) return HMG_EINVAL;
  Dev dg(db->device);
  return cuda_status(cudaMemcpyAsync(db->d_words, image, (size_t)hmg_db_packed_bytes(db), cudaMemcpyHostToDevice,
                                     (cudaStream_t)stream));
}

void hmg_db_destroy(hmg_db* db) {
  if (!db) return;
  if (db->device >= 0) {
    Dev dg(db->device);
    cudaFree(db->d_words);
    cudaFree(db->d_woff16);
    cudaFree(db->d_len);
    cudaFree(db->d_order);
    cudaFree(db->d_inv);
    cudaFree(db->d_tjb);
    cudaFree(db->d_move);
    cudaFree(db->d_chunk_start);
    cudaGetLastError();
  }
  delete db;
}

hmg_status hmg_msv(const hmg_profile* pc, const hmg_db* db, double F1, void* stream, uint8_t* raw, uint8_t* pass) {
  hmg_profile* p = const_cast<hmg_profile*>(pc);
  if (!p || !db || (!raw && db->nseq) || p->device != db->device || db->device < 0) return HMG_EINVAL;
  if (pass && (!p->has_ev || !(F1 > 0.0 && F1 <= 1.0))) return HMG_EINVAL;
  if (db->nseq == 0) return HMG_OK;
  Dev dg(db->device);
  cudaStream_t st = (cudaStream_t)stream;
  const uint16_t* thr = nullptr;
  if (pass) {
    hmg_status s = msv_thr_table(p, db, F1, &thr, st);
    if (s != HMG_OK) return s;
  }
  cudaError_t e = cudaSuccess;
  hmg_status s;
  {
    Scratch S(st);
    auto* raw_sorted = (uint8_t*)S.get((size_t)db->nseq, &e);
    void* tmp = S.get(scan_tmp_bytes(db->nseq) + (size_t)db->nseq + 16, &e);
    if (e) return cuda_status(e);
    mark_reset();
    s = run_msv(p, db, st, raw_sorted, S);
    if (s != HMG_OK) return s;
    e = msv_finish(raw_sorted, db->d_len, db->d_order, db->nseq, thr, raw, pass, nullptr, nullptr, nullptr, tmp,
                   st);
    mark(3, st);
  }
  if (e == cudaSuccess) e = cudaGetLastError();
  return cuda_status(e);
}

hmg_status hmg_viterbi(const hmg_profile* pc, const hmg_db* db, const int32_t* ids, int64_t n, double F2,
                       void* stream, int16_t* raw, uint8_t* pass) {
  hmg_profile* p = const_cast<hmg_profile*>(pc);
  if (!p || !db || !p->has_tsc || (!raw && db->nseq) || p->device != db->device || db->device < 0)
    return HMG_EINVAL;
  if (pass && (!p->has_ev || !(F2 > 0.0 && F2 <= 1.0))) return HMG_EINVAL;
  if (ids && n < 0) return HMG_EINVAL;
  if (db->nseq == 0 || (ids && n == 0)) return HMG_OK;
  Dev dg(db->device);
  cudaStream_t st = (cudaStream_t)stream;
  const int32_t* thr = nullptr;
  if (pass) {
    hmg_status s = vit_thr_table(p, db, F2, &thr, st);
    if (s != HMG_OK) return s;
  }
  cudaError_t e = cudaSuccess;
  {
    Scratch S(st);
    auto* raw_sorted = (int16_t*)S.get(sizeof(int16_t) * (size_t)db->nseq, &e);
    if (e) return cuda_status(e);
    const int32_t* list = nullptr;
    const int64_t* nl = nullptr;
    int64_t nmax = db->nseq;
    if (ids) {
      auto* sl = (int32_t*)S.get(sizeof(int32_t) * (size_t)n, &e);
      auto* cnt = (int64_t*)S.get(sizeof(int64_t), &e);
      if (e) return cuda_status(e);
      if ((e = to_sorted_ids(ids, n, db->d_inv, sl, st))) return cuda_status(e);
      if ((e = set_count(cnt, n, st))) return cuda_status(e);
      list = sl;
      nl = cnt;
      nmax = n;
    }
    mark_reset();
    hmg_status s = run_vit(p, db, list, nl, st, raw_sorted, S, nullptr, 0, true, nmax);
    if (s != HMG_OK) return s;
    e = vit_finish(raw_sorted, list, nl, nmax, db->d_len, db->d_order, thr, raw, pass, nullptr, st);
    mark(5, st);
  }
  if (e == cudaSuccess) e = cudaGetLastError();
  return cuda_status(e);
}

static cudaStream_t* side_streams(int device);

// h_image (optional): pinned host copy of the packed DB image (hmg_db_image); it is uploaded in
// kUploadParts length-ordered parts on a side stream while the MSV kernel scores the parts that
// have landed (one launch per part), so the H2D overlaps the filter.
constexpr int kUploadParts = 12;    // capacity; parts used: tuning UPLOAD_PARTS (default 6)

// Joins side streams back into the caller's stream on every exit path of a call that forked
// them (declared after the call's Scratch, so it runs first and the scratch is freed on `st`
// only after the side-stream work that uses it), and destroys the call's events.
struct SideJoin {
  cudaStream_t st;
  std::vector<cudaStream_t> side;
  std::vector<cudaEvent_t> events;
  explicit SideJoin(cudaStream_t s) : st(s) {}
  void add(cudaStream_t s) {
    if (s && s != st && std::find(side.begin(), side.end(), s) == side.end()) side.push_back(s);
  }
  ~SideJoin() {
    for (cudaStream_t s : side) {
      cudaEvent_t ev = nullptr;
      if (cudaEventCreateWithFlags(&ev, cudaEventDisableTiming) == cudaSuccess) {
        if (cudaEventRecord(ev, s) == cudaSuccess) cudaStreamWaitEvent(st, ev, 0);
        cudaEventDestroy(ev);
      }
    }
    for (cudaEvent_t ev : events)
      if (ev) cudaEventDestroy(ev);
  }
};

static hmg_status pipeline_impl(const hmg_profile* pc, const hmg_db* db, double F1, double F2, void* stream,
                                uint8_t* msv_raw, int16_t* vit_raw, uint8_t* flags, int32_t* survivor_ids,
                                int64_t* n_survivors, uint8_t* vpass_sorted, const uint32_t* h_image = nullptr) {
  hmg_profile* p = const_cast<hmg_profile*>(pc);
  if (!p || !db || !p->has_tsc || !p->has_ev || p->device != db->device || db->device < 0) return HMG_EINVAL;
  if (!(F1 > 0.0 && F1 <= 1.0) || !(F2 > 0.0 && F2 <= 1.0)) return HMG_EINVAL;
  if (db->nseq && (!msv_raw || !vit_raw || !flags || !survivor_ids || !n_survivors)) return HMG_EINVAL;
  Dev dg(db->device);
  cudaStream_t st = (cudaStream_t)stream;
  if (db->nseq == 0) return n_survivors ? cuda_status(set_count(n_survivors, 0, st)) : HMG_OK;
  const uint16_t* tm = nullptr;
  const int32_t* tv = nullptr;
  hmg_status s = msv_thr_table(p, db, F1, &tm, st);
  if (s == HMG_OK) s = vit_thr_table(p, db, F2, &tv, st);
  if (s != HMG_OK) return s;
  cudaError_t e = cudaSuccess;
  {
    Scratch S(st);
    const int64_t n = db->nseq;
    auto* raw_sorted = (uint8_t*)S.get((size_t)n, &e);
    auto* vraw_sorted = (int16_t*)S.get(sizeof(int16_t) * (size_t)n, &e);
    auto* surv = (int32_t*)S.get(sizeof(int32_t) * (size_t)n, &e);
    void* tmp = S.get(scan_tmp_bytes(n) + (size_t)n + 16, &e);
    if (e) return cuda_status(e);
    mark_reset();
    // pipeline long lane (long.cu): chunked MSV of the longest sequences on the whole GPU, then
    // their Viterbi filter on SMs held alone by pipe_long_vit_kernel while the main MSV kernel
    // (programmatic dependent launch) fills the other SMs
    const int64_t nlong = (p->long_QV > 0 && msv_fast_on(p, db) &&
                           (p->long_pair || (!p->vit_generic && p->vit_W == 0)) &&
                           !tune_int("NO_LONG_LANE", 0)) ? db->nlong : 0;
    uint8_t* owned = nullptr;
    // work-queue counters (2 per upload part)
    auto* mctr = (unsigned long long*)S.get(sizeof(unsigned long long) * 2 * kUploadParts, &e);
    if (e) return cuda_status(e);
    if ((e = cudaMemsetAsync(mctr, 0, sizeof(unsigned long long) * 2 * kUploadParts, st))) return cuda_status(e);
    // overlapped upload: part boundaries (sorted indices), part 0 >= the long lane; part k's
    // words are one contiguous run of the image
    int64_t bnd[kUploadParts + 1] = {0};
    int nparts = 1;
    bnd[1] = n;
    cudaEvent_t up_ev[kUploadParts] = {};
    cudaStream_t cs = nullptr;
    SideJoin join(st);                              // every exit: side streams joined into st
    if (h_image) {
      nparts = std::max(2, std::min(kUploadParts, tune_int("UPLOAD_PARTS", 5)));   // profiles/e2e_r02zza.jsonl
      // a small first part (the filter waits for it; later parts land faster than MSV consumes
      // them), then equal parts of the rest
      const int first_pm = tune_int("UPLOAD_FIRST_PERMILLE", 50);   // profiles/upload_parts_r01b.jsonl
      // the rest in parts whose sizes follow a geometric ratio HMG_UPLOAD_GROW / 1000 (1000 = equal
      // parts); a ratio below 1 shrinks the last parts, whose MSV cannot start before they land
      const int64_t r0 = db->residues * first_pm / 1000;
      const double g = std::max(1, tune_int("UPLOAD_GROW", 1000)) / 1000.0;
      double cut[kUploadParts] = {0.0}, wsum = 0.0, wk = 1.0;
      for (int q = 1; q < nparts; ++q, wk *= g) wsum += wk;
      wk = 1.0;
      for (int q = 1; q < nparts; ++q, wk *= g)
        cut[q] = (q > 1 ? cut[q - 1] : (double)r0) + (double)(db->residues - r0) * wk / wsum;
      int64_t acc = 0, k = 1;
      for (int64_t j = 0; j < n && k < nparts; ++j) {
        acc += db->len_sorted[j];
        if ((k == 1 ? acc >= r0 : (double)acc >= cut[k - 1]) && j + 1 >= nlong) bnd[k++] = j + 1;
      }
      while (k < nparts) bnd[k++] = n;
      bnd[nparts] = n;
      cudaStream_t* side = side_streams(db->device);
      if (!side) return HMG_ECUDA;
      cs = side[0];
      join.add(cs);
      cudaEvent_t fork = nullptr;
      if ((e = cudaEventCreateWithFlags(&fork, cudaEventDisableTiming))) return cuda_status(e);
      if ((e = cudaEventRecord(fork, st)) || (e = cudaStreamWaitEvent(cs, fork, 0))) return cuda_status(e);
      cudaEventDestroy(fork);
      const int64_t nw_all = std::max<int64_t>(db->nwords, 4);
      for (int q = 0; q < nparts; ++q) {
        const int64_t w0 = bnd[q] < n ? (int64_t)db->woff16_h[bnd[q]] * 4 : nw_all;
        const int64_t w1 = bnd[q + 1] < n ? (int64_t)db->woff16_h[bnd[q + 1]] * 4 : nw_all;
        if ((e = cudaEventCreateWithFlags(&up_ev[q], cudaEventDisableTiming))) return cuda_status(e);
        join.events.push_back(up_ev[q]);
        if (w1 > w0 && (e = cudaMemcpyAsync(db->d_words + w0, h_image + w0, (size_t)(w1 - w0) * 4,
                                            cudaMemcpyHostToDevice, cs)))
          return cuda_status(e);
        if ((e = cudaEventRecord(up_ev[q], cs))) return cuda_status(e);
      }
      if ((e = cudaStreamWaitEvent(st, up_ev[0], 0))) return cuda_status(e);
    }
    // the parts' MSV kernels run on a second side stream (they never read the long lane's
    // sequences), so the long lane's exclusive-SM Viterbi overlaps all of them
    // consecutive parts' MSV kernels rotate over nms side streams, so a part's kernel starts on the
    // SMs the previous part's tail frees (UPLOAD_MSV_STREAMS, 1..4)
    constexpr int kMaxMsvStreams = 4;
    cudaStream_t ms = st;
    cudaStream_t mss[kMaxMsvStreams] = {st, st, st, st};
    cudaEvent_t ms_done[kMaxMsvStreams] = {};
    const bool overlap = h_image && msv_fast_on(p, db);
    const int nms = overlap ? std::max(1, std::min(kMaxMsvStreams, tune_int("UPLOAD_MSV_STREAMS", 2))) : 1;
    if (h_image && !overlap) {                      // exact-kernel profiles: plain upload first
      for (int q = 1; q < nparts; ++q)
        if ((e = cudaStreamWaitEvent(st, up_ev[q], 0))) return cuda_status(e);
    }
    if (overlap) {
      cudaEvent_t f2 = nullptr;
      if ((e = cudaEventCreateWithFlags(&f2, cudaEventDisableTiming))) return cuda_status(e);
      if ((e = cudaEventRecord(f2, st))) return cuda_status(e);
      for (int k = 0; k < nms; ++k) {
        mss[k] = side_streams(db->device)[1 + k];
        join.add(mss[k]);
        if ((e = cudaStreamWaitEvent(mss[k], f2, 0))) return cuda_status(e);
        if ((e = cudaEventCreateWithFlags(&ms_done[k], cudaEventDisableTiming))) return cuda_status(e);
        join.events.push_back(ms_done[k]);
      }
      cudaEventDestroy(f2);
      ms = mss[0];
    }
    mark(0, st);
    if (nlong > 0) {
      LongArgs la{};
      if ((s = run_msv_long_chunks(p, db, st, raw_sorted, S, &la)) != HMG_OK) return s;
      owned = la.owned;
      la.v.words = db->d_words;
      la.v.woff16 = db->d_woff16;
      la.v.len = db->d_len;
      la.v.nseq = n;
      la.v.move = db->d_move;
      // (pair lane: the pair kernel's tables when it runs whole warps, else the long lane's own)
      const bool own = p->d_long_rsc != nullptr;
      la.v.rsc = reinterpret_cast<const int16_t*>(p->long_pair && !own ? (void*)p->d_pair_rsc : (void*)p->d_long_rsc);
      la.v.tr = reinterpret_cast<const int32_t*>(p->long_pair && !own ? (void*)p->d_pair_tr : (void*)p->d_long_tr);
      la.v.tbm_min = p->tbm_min;
      la.v.safe = 32767 - p->rmax;
      la.v.M = p->M;
      la.v.raw_sorted = vraw_sorted;
      la.thr = tm;
      // blocks (SMs) for the long-survivor Viterbi: about one per 20 long sequences, 2..16
      int nb = (int)std::min<int64_t>(std::max<int64_t>((nlong + 19) / 20, 2), 16);
      nb = tune_int("PIPE_LONG_SMS", nb);
      int ok = 0;
      if ((e = launch_pipe_long_vit(p->long_QV, p->long_pair, la, nb, st, &ok))) return cuda_status(e);
      if (!ok) return HMG_EUNSUPPORTED;
    }
    if (!overlap) {
      s = run_msv_fast(p, db, st, raw_sorted, S, nlong > 0 ? nlong : -1, nlong > 0, false, mctr);   // Fig 1: MSV
      if (s != HMG_OK) return s;
    } else {
      for (int q = 0; q < nparts; ++q) {          // MSV of each part once it has landed
        cudaStream_t mq = mss[q % nms];
        if ((e = cudaStreamWaitEvent(mq, up_ev[q], 0))) return cuda_status(e);
        const int64_t lo = std::max(bnd[q], nlong), hi = bnd[q + 1];
        if (hi > lo) {
          s = run_msv_fast(p, db, mq, raw_sorted, S, lo, false, false, mctr + 2 * q, hi);
          if (s != HMG_OK) return s;
        }
      }
      for (int k = 0; k < nms; ++k)
        if ((e = cudaEventRecord(ms_done[k], mss[k])) || (e = cudaStreamWaitEvent(st, ms_done[k], 0)))
          return cuda_status(e);
    }
    s = run_msv_redo(p, db, st, raw_sorted, S);
    if (s != HMG_OK) return s;
    e = msv_finish(raw_sorted, db->d_len, db->d_order, n, tm, msv_raw, flags, surv, n_survivors, survivor_ids, tmp,
                   st);                                                       // pass + compaction
    if (e) return cuda_status(e);
    s = run_vit(p, db, surv, n_survivors, st, vraw_sorted, S, owned, nlong);  // P7Viterbi on survivors
    if (s != HMG_OK) return s;

    e = vit_finish(vraw_sorted, surv, n_survivors, n, db->d_len, db->d_order, tv, vit_raw, nullptr, flags, st,
                   vpass_sorted);
    mark(5, st);
  }
  if (e == cudaSuccess) e = cudaGetLastError();
  return cuda_status(e);
}


hmg_status hmg_pipeline(const hmg_profile* p, const hmg_db* db, double F1, double F2, void* stream,
                        uint8_t* msv_raw, int16_t* vit_raw, uint8_t* flags, int32_t* survivor_ids,
                        int64_t* n_survivors) {
  return pipeline_impl(p, db, F1, F2, stream, msv_raw, vit_raw, flags, survivor_ids, n_survivors, nullptr);
}

hmg_status hmg_pipeline_upload(const hmg_profile* p, hmg_db* db, const uint32_t* image, double F1, double F2,
                               void* stream, uint8_t* msv_raw, int16_t* vit_raw, uint8_t* flags,
                               int32_t* survivor_ids, int64_t* n_survivors) {
  if (!db || !image || db->device < 0) return HMG_EINVAL;
  return pipeline_impl(p, db, F1, F2, stream, msv_raw, vit_raw, flags, survivor_ids, n_survivors, nullptr, image);
}

// Forward stage over a sorted-order list (device list + device count, nmax = list capacity).
static hmg_status run_fwd(const hmg_profile* p, const hmg_db* db, const int32_t* list, const int64_t* nlist,
                          cudaStream_t st, float* nats, uint8_t* flags, Scratch& S) {
  if (p->fwd_W == 0) return HMG_EUNSUPPORTED;
  cudaError_t e = cudaSuccess;
  auto* ctr = (unsigned long long*)S.get(sizeof(unsigned long long), &e);
  if (e) return cuda_status(e);
  if ((e = cudaMemsetAsync(ctr, 0, sizeof(unsigned long long), st))) return cuda_status(e);
  FwdArgs a{};
  a.words = db->d_words;
  a.woff16 = db->d_woff16;
  a.len = db->d_len;
  a.order = db->d_order;
  a.list = list;
  a.nlist = nlist;
  a.nseq = db->nseq;
  a.etab = p->d_fwd_e;
  a.tr = p->d_fwd_t;
  a.cst = p->d_fwd_c;
  a.rows_smem = p->fwd_rows;
  a.out = nats;
  a.flags = flags;
  a.counter = ctr;
  int ok = 0;
  if ((e = launch_fwd(p->fwd_T, p->fwd_Q, p->fwd_S, p->fwd_rows, a, st, &ok))) return cuda_status(e);
  return ok ? HMG_OK : HMG_EUNSUPPORTED;
}

hmg_status hmg_forward(const hmg_profile* pc, const hmg_db* db, const int32_t* ids, int64_t n, void* stream,
                       float* nats) {
  hmg_profile* p = const_cast<hmg_profile*>(pc);
  if (!p || !db || !p->has_tsc || (!nats && db->nseq) || p->device != db->device || db->device < 0)
    return HMG_EINVAL;
  if (ids && n < 0) return HMG_EINVAL;
  if (p->fwd_W == 0 || p->msc_max > kFwdMscMax) return HMG_EUNSUPPORTED;
  if (db->nseq == 0 || (ids && n == 0)) return HMG_OK;
  Dev dg(db->device);
  cudaStream_t st = (cudaStream_t)stream;
  cudaError_t e = cudaSuccess;
  hmg_status s;
  {
    Scratch S(st);
    const int32_t* list = nullptr;
    const int64_t* nl = nullptr;
    if (ids) {
      auto* sl = (int32_t*)S.get(sizeof(int32_t) * (size_t)n, &e);
      auto* cnt = (int64_t*)S.get(sizeof(int64_t), &e);
      if (e) return cuda_status(e);
      if ((e = to_sorted_ids(ids, n, db->d_inv, sl, st))) return cuda_status(e);
      if ((e = set_count(cnt, n, st))) return cuda_status(e);
      list = sl;
      nl = cnt;
    }
    mark_reset();
    mark(5, st);
    s = run_fwd(p, db, list, nl, st, nats, nullptr, S);
    mark(6, st);
  }
  if (s != HMG_OK) return s;
  return cuda_status(cudaGetLastError());
}

hmg_status hmg_pipeline_forward(const hmg_profile* pc, const hmg_db* db, double F1, double F2, void* stream,
                                uint8_t* msv_raw, int16_t* vit_raw, uint8_t* flags, int32_t* survivor_ids,
                                int64_t* n_survivors, float* fwd_nats, int32_t* fwd_ids, int64_t* n_fwd) {
  hmg_profile* p = const_cast<hmg_profile*>(pc);
  if (!p || !db || p->device != db->device || db->device < 0) return HMG_EINVAL;
  if (db->nseq && (!fwd_nats || !fwd_ids || !n_fwd)) return HMG_EINVAL;
  if (p->has_tsc && (p->fwd_W == 0 || p->msc_max > kFwdMscMax)) return HMG_EUNSUPPORTED;
  Dev dg(db->device);
  cudaStream_t st = (cudaStream_t)stream;
  const int64_t n = db->nseq;
  cudaError_t e = cudaSuccess;
  hmg_status s;
  {
    Scratch S(st);
    auto* vpass = (uint8_t*)S.get((size_t)std::max<int64_t>(n, 1), &e);
    auto* fl = (int32_t*)S.get(sizeof(int32_t) * (size_t)std::max<int64_t>(n, 1), &e);
    void* tmp = S.get(scan_tmp_bytes(n) + 16, &e);
    if (e) return cuda_status(e);
    if (n && (e = cudaMemsetAsync(vpass, 0, (size_t)n, st))) return cuda_status(e);
    s = pipeline_impl(p, db, F1, F2, stream, msv_raw, vit_raw, flags, survivor_ids, n_survivors, vpass);
    if (s != HMG_OK) return s;
    if (n == 0) return n_fwd ? cuda_status(set_count(n_fwd, 0, st)) : HMG_OK;
    // Viterbi passes -> Forward list (stable, schedule order) -> Forward kernel (Fig 1)
    if ((e = compact_flags(vpass, n, db->d_order, fl, fwd_ids, n_fwd, tmp, st))) return cuda_status(e);
    s = run_fwd(p, db, fl, n_fwd, st, fwd_nats, flags, S);
    mark(6, st);
  }
  if (s != HMG_OK) return s;
  return cuda_status(cudaGetLastError());
}

// ------------------------------------------------------------------ many-profile MSV (f4)
constexpr int kSideStreams = 8;

// Per-device pool of non-blocking side streams (created on first use, kept for the process).
static cudaStream_t* side_streams(int device) {
  static std::mutex mu;
  static std::vector<std::vector<cudaStream_t>> pools;
  std::lock_guard<std::mutex> g(mu);
  if ((int)pools.size() <= device) pools.resize(device + 1);
  auto& v = pools[device];
  if (v.empty()) {
    for (int k = 0; k < kSideStreams; ++k) {
      cudaStream_t s = nullptr;
      if (cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking) != cudaSuccess) {
        cudaGetLastError();
        for (auto x : v) cudaStreamDestroy(x);
        v.clear();
        return nullptr;
      }
      v.push_back(s);
    }
  }
  return v.data();
}

// Striped table of profile p in lane geometry (G, Q): its own table when the geometry matches,
// else built on first use and cached in the profile (guarded by its mutex).
static hmg_status msv_table_for(hmg_profile* p, int G, int Q, const uint32_t** out) {
  if (G == p->msv_G && Q == p->msv_Q && p->d_msv_prof) {
    *out = p->d_msv_prof;
    return HMG_OK;
  }
  std::lock_guard<std::mutex> g(p->mu);
  for (auto& t : p->msv_tabs)
    if (t.G == G && t.Q == Q) {
      *out = t.d;
      return HMG_OK;
    }
  auto h = msv_table(*p, G, Q);
  uint32_t* d = nullptr;
  hmg_status s = upload(&d, h.data(), h.size());
  if (s != HMG_OK) return s;
  p->msv_tabs.push_back({G, Q, d});
  *out = d;
  return HMG_OK;
}

// Outputs of the batched pipeline tail (hmg_pipeline_batch): per-profile rows of [nprof][nseq].
struct BatchTail {
  double F2;
  int16_t* vit_raw;
  uint8_t* flags;
  int32_t* survivor_ids;
  int64_t* n_survivors;
  float* fwd_nats;           // optional Forward stage (all three or none)
  int32_t* fwd_ids;
  int64_t* n_fwd;
};

static hmg_status msv_batch_impl(const hmg_profile* const* profs, int nprof, const hmg_db* db, double F1,
                                 void* stream, uint8_t* raw, uint8_t* pass, const BatchTail* tail) {
  if (!profs || nprof < 1 || nprof > 65535 || !db || db->device < 0 || (!raw && db->nseq)) return HMG_EINVAL;
  if ((pass || tail) && !(F1 > 0.0 && F1 <= 1.0)) return HMG_EINVAL;
  for (int i = 0; i < nprof; ++i) {
    if (!profs[i] || profs[i]->device != db->device) return HMG_EINVAL;
    if ((pass || tail) && !profs[i]->has_ev) return HMG_EINVAL;
    if (tail && !profs[i]->has_tsc) return HMG_EINVAL;
    if (tail && tail->fwd_nats && (profs[i]->fwd_W == 0 || profs[i]->msc_max > kFwdMscMax)) return HMG_EUNSUPPORTED;
  }
  if (db->nseq == 0) {
    if (tail && tail->n_survivors) {
      cudaError_t e0 = cudaMemsetAsync(tail->n_survivors, 0, sizeof(int64_t) * nprof, (cudaStream_t)stream);
      if (e0 == cudaSuccess && tail->n_fwd)
        e0 = cudaMemsetAsync(tail->n_fwd, 0, sizeof(int64_t) * nprof, (cudaStream_t)stream);
      return cuda_status(e0);
    }
    return HMG_OK;
  }
  Dev dg(db->device);
  cudaStream_t st = (cudaStream_t)stream;
  const int64_t n = db->nseq;
  // buckets: profiles sorted by M (descending); a bucket takes the geometry of its largest model
  // and every following profile whose own register count at that G is >= (100 - pad)% of it
  // (padding waste <= pad%); profiles outside the fast kernel's precondition go to the exact
  // pair kernel
  std::vector<int> idx;
  std::vector<int> slow;
  for (int i = 0; i < nprof; ++i) {
    hmg_profile* p = const_cast<hmg_profile*>(profs[i]);
    // (the bucket geometry is chosen below: the int8-chunk bound is required of every fast profile)
    if (p->msv_fast && p->msv_Q > 0 && msv_byte_exact(tjb_of(std::max(db->Lmax, 0)), p->tbm, p->bias))
      idx.push_back(i);
    else slow.push_back(i);
  }
  std::stable_sort(idx.begin(), idx.end(), [&](int a, int b) { return profs[a]->M > profs[b]->M; });
  struct Bucket { int G, Q, r0, r1; };
  std::vector<Bucket> buckets;
  std::vector<int> rows;                        // row r of the raw matrix -> caller profile index
  // (measured, profiles/batch_bench_r01.jsonl: padding pays on small DBs -- fewer, fuller
  //  launches -- and costs ~5% of cells on large ones, where every bucket fills the GPU anyway)
  const bool large = n >= 50000;
  const int pad_pct = tune_int("MSV_BATCH_PAD", large ? 0 : 20);
  for (size_t j = 0; j < idx.size();) {
    int G = 0, Q = 0;
    msv_geometry(profs[idx[j]]->M, &G, &Q);
    const int r0 = (int)rows.size();
    while (j < idx.size()) {
      const int qj = (profs[idx[j]]->M + (kMsvQPlus1 ? 1 : 0) + 2 * G - 1) / (2 * G);
      if ((int)rows.size() > r0 && 100 * qj < (100 - pad_pct) * Q) break;
      rows.push_back(idx[j]);
      ++j;
    }
    buckets.push_back({G, Q, r0, (int)rows.size()});
  }
  const int nfast = (int)rows.size();
  for (int i : slow) rows.push_back(i);
  // per-row arrays (bucket order)
  std::vector<const uint32_t*> tabs(nprof, nullptr);
  std::vector<const uint8_t*> costs(nprof);
  std::vector<const uint16_t*> thr(nprof, nullptr);
  std::vector<int> Ms(nprof), bias(nprof), tbm(nprof);
  int Mmax = 0;
  for (int r = 0; r < nprof; ++r) {
    hmg_profile* p = const_cast<hmg_profile*>(profs[rows[r]]);
    costs[r] = p->d_cost;
    Ms[r] = p->M;
    bias[r] = p->bias;
    tbm[r] = p->tbm;
    Mmax = std::max(Mmax, p->M);
    if (pass || tail) {
      hmg_status s = msv_thr_table(p, db, F1, &thr[r], st);
      if (s != HMG_OK) return s;
    }
  }
  for (const auto& b : buckets)
    for (int r = b.r0; r < b.r1; ++r) {
      hmg_status s = msv_table_for(const_cast<hmg_profile*>(profs[rows[r]]), b.G, b.Q, &tabs[r]);
      if (s != HMG_OK) return s;
    }
  cudaError_t e = cudaSuccess;
  {
    Scratch S(st);
    auto* raw_sorted = (uint8_t*)S.get((size_t)nprof * (size_t)n, &e);
    auto* d_tabs = (const uint32_t**)S.get(sizeof(void*) * nprof, &e);
    auto* d_costs = (const uint8_t**)S.get(sizeof(void*) * nprof, &e);
    auto* d_thr = (const uint16_t**)S.get(sizeof(void*) * nprof, &e);
    auto* d_ints = (int*)S.get(sizeof(int) * 4 * nprof, &e);
    auto* list = (int64_t*)S.get(sizeof(int64_t) * (size_t)nprof * (size_t)n, &e);
    auto* cnt = (int64_t*)S.get(sizeof(int64_t), &e);
    const int nwarps_exact = 148 * 16;
    auto* scr = (uint8_t*)S.get((size_t)nwarps_exact * 2 * (Mmax + 1), &e);
    if (e) return cuda_status(e);
    std::vector<int> ints;
    ints.insert(ints.end(), Ms.begin(), Ms.end());
    ints.insert(ints.end(), bias.begin(), bias.end());
    ints.insert(ints.end(), tbm.begin(), tbm.end());
    ints.insert(ints.end(), rows.begin(), rows.end());
    if ((e = cudaMemcpyAsync(d_tabs, tabs.data(), sizeof(void*) * nprof, cudaMemcpyHostToDevice, st)) ||
        (e = cudaMemcpyAsync(d_costs, costs.data(), sizeof(void*) * nprof, cudaMemcpyHostToDevice, st)) ||
        (e = cudaMemcpyAsync(d_thr, thr.data(), sizeof(void*) * nprof, cudaMemcpyHostToDevice, st)) ||
        (e = cudaMemcpyAsync(d_ints, ints.data(), sizeof(int) * 4 * nprof, cudaMemcpyHostToDevice, st)))
      return cuda_status(e);
    const int* d_M = d_ints;
    const int* d_bias = d_ints + nprof;
    const int* d_tbm = d_ints + 2 * nprof;
    const int* d_rows = d_ints + 3 * nprof;
    if (nfast < nprof &&   // profiles outside the fast precondition: every pair to the exact kernel
        (e = cudaMemsetAsync(raw_sorted + (size_t)nfast * n, 254, (size_t)(nprof - nfast) * n, st)))
      return cuda_status(e);
    mark_reset();
    mark(0, st);
    auto* ctr = (unsigned long long*)S.get(sizeof(unsigned long long) * std::max<size_t>(buckets.size(), 1), &e);
    if (e) return cuda_status(e);
    if ((e = cudaMemsetAsync(ctr, 0, sizeof(unsigned long long) * std::max<size_t>(buckets.size(), 1), st)))
      return cuda_status(e);
    // buckets run concurrently on a pool of side streams (forked from and joined back into st), so
    // one bucket's tail -- its longest sequences -- overlaps the other buckets' work
    const int nside = (int)std::min<size_t>(buckets.size(), kSideStreams);
    cudaStream_t* side = nside > 1 ? side_streams(db->device) : nullptr;
    if (nside > 1 && !side) return HMG_ECUDA;
    cudaEvent_t fork = nullptr, join[kSideStreams] = {};
    if (nside > 1) {
      if ((e = cudaEventCreateWithFlags(&fork, cudaEventDisableTiming))) return cuda_status(e);
      if ((e = cudaEventRecord(fork, st))) return cuda_status(e);
      for (int k = 0; k < nside; ++k) {
        if ((e = cudaStreamWaitEvent(side[k], fork, 0))) return cuda_status(e);
        if ((e = cudaEventCreateWithFlags(&join[k], cudaEventDisableTiming))) return cuda_status(e);
      }
    }
    for (size_t bi = 0; bi < buckets.size(); ++bi) {
      const Bucket& b = buckets[bi];
      cudaStream_t bs = nside > 1 ? side[bi % nside] : st;
      MsvMultiArgs m{};
      m.base = msv_args(profs[rows[b.r0]], db);
      m.nprof = b.r1 - b.r0;
      m.prof = d_tabs + b.r0;
      m.bias = d_bias + b.r0;
      m.tbm = d_tbm + b.r0;
      m.raw = raw_sorted + (size_t)b.r0 * n;
      // chunk = R rounds of the block's 8 warps x 32/G sequences: large R keeps the item-boundary
      // idling of a block's warps small (large DBs), R = 4 measured best on config-1-sized DBs
      const int per_round = (32 / b.G) * 8;
      const int R = tune_int("MSV_BATCH_ROUNDS", large ? 16 : 4);
      m.chunk = per_round * R;
      m.nchunks = (n + m.chunk - 1) / m.chunk;
      m.counter = ctr + bi;
      int ok = 0;
      if ((e = launch_msv_multi(b.G, b.Q, m, bs, &ok))) return cuda_status(e);
      if (!ok) return HMG_EUNSUPPORTED;
    }
    if (nside > 1) {
      for (int k = 0; k < nside; ++k) {
        if ((e = cudaEventRecord(join[k], side[k]))) return cuda_status(e);
        if ((e = cudaStreamWaitEvent(st, join[k], 0))) return cuda_status(e);
        cudaEventDestroy(join[k]);
      }
      cudaEventDestroy(fork);
    }
    mark(1, st);
    // exact re-score of the flagged pairs
    if ((e = select_redo_pairs(raw_sorted, (int64_t)nprof * n, list, cnt, st))) return cuda_status(e);
    MsvPairArgs x{};
    x.words = db->d_words;
    x.woff16 = db->d_woff16;
    x.len = db->d_len;
    x.nseq = n;
    x.tjb = db->d_tjb;
    x.cost = d_costs;
    x.M = d_M;
    x.bias = d_bias;
    x.tbm = d_tbm;
    x.list = list;
    x.nlist = cnt;
    x.raw = raw_sorted;
    x.scratch = scr;
    x.Mmax = Mmax;
    if ((e = launch_msv_pairs_exact(x, nwarps_exact, st))) return cuda_status(e);
    mark(2, st);
    if (!tail) {
      e = msv_flags_multi(raw_sorted, nprof, db->d_len, db->d_order, n, pass ? d_thr : nullptr, d_rows, raw, pass,
                          st);
      mark(3, st);
    } else {
      // Fig 1 per profile: pass flags of every row and the stable survivor compaction of every row
      // in four launches on st, then each profile's Viterbi filter on its survivors; the profiles'
      // Viterbi chains run concurrently on the side streams
      auto* fs = (uint8_t*)S.get((size_t)nprof * (size_t)n, &e);
      auto* surv_all = (int32_t*)S.get(sizeof(int32_t) * (size_t)nprof * (size_t)n, &e);
      void* ctmp = S.get(compact_rows_tmp_bytes(n, nprof), &e);
      if (e) return cuda_status(e);
      if ((e = msv_flags_multi(raw_sorted, nprof, db->d_len, db->d_order, n, d_thr, d_rows, raw, tail->flags, st,
                               fs)))
        return cuda_status(e);
      if ((e = compact_rows(fs, nprof, n, db->d_order, surv_all, tail->survivor_ids, tail->n_survivors, d_rows, ctmp,
                            st)))
        return cuda_status(e);
      std::vector<const int32_t*> tv(nprof);
      for (int r = 0; r < nprof; ++r) {
        hmg_status s = vit_thr_table(const_cast<hmg_profile*>(profs[rows[r]]), db, tail->F2, &tv[r], st);
        if (s != HMG_OK) return s;
      }
      const int ns = std::min(nprof, kSideStreams);
      cudaStream_t* side = ns > 1 ? side_streams(db->device) : nullptr;
      if (ns > 1 && !side) return HMG_ECUDA;
      cudaEvent_t fork = nullptr, join[kSideStreams] = {};
      if (ns > 1) {
        if ((e = cudaEventCreateWithFlags(&fork, cudaEventDisableTiming))) return cuda_status(e);
        if ((e = cudaEventRecord(fork, st))) return cuda_status(e);
        for (int k = 0; k < ns; ++k) {
          if ((e = cudaStreamWaitEvent(side[k], fork, 0))) return cuda_status(e);
          if ((e = cudaEventCreateWithFlags(&join[k], cudaEventDisableTiming))) return cuda_status(e);
        }
      }
      {
        std::vector<Scratch*> SS;
        struct Bufs { int16_t* vraw; void* tmp; uint8_t* vpass; int32_t* fl; };
        std::vector<Bufs> B;
        hmg_status s = HMG_OK;
        for (int k = 0; k < std::max(ns, 1); ++k) {
          cudaStream_t sk = ns > 1 ? side[k] : st;
          SS.push_back(new Scratch(sk));
          Bufs b{};
          b.vraw = (int16_t*)SS.back()->get(sizeof(int16_t) * (size_t)n, &e);
          b.tmp = SS.back()->get(scan_tmp_bytes(n) + (size_t)n + 16, &e);
          if (tail->fwd_nats) {
            b.vpass = (uint8_t*)SS.back()->get((size_t)n, &e);
            b.fl = (int32_t*)SS.back()->get(sizeof(int32_t) * (size_t)n, &e);
          }
          B.push_back(b);
        }
        for (int r = 0; r < nprof && !e && s == HMG_OK; ++r) {
          const int k = ns > 1 ? r % ns : 0;
          cudaStream_t sk = ns > 1 ? side[k] : st;
          const int i = rows[r];
          const hmg_profile* pi = profs[i];
          const size_t ro = (size_t)i * n;
          const int32_t* surv = surv_all + (size_t)r * n;
          s = run_vit(pi, db, surv, tail->n_survivors + i, sk, B[k].vraw, *SS[k], nullptr, 0, false, n);
          if (s != HMG_OK) break;
          if (tail->fwd_nats && (e = cudaMemsetAsync(B[k].vpass, 0, (size_t)n, sk))) break;
          e = vit_finish(B[k].vraw, surv, tail->n_survivors + i, n, db->d_len, db->d_order, tv[r],
                         tail->vit_raw + ro, nullptr, tail->flags + ro, sk, tail->fwd_nats ? B[k].vpass : nullptr);
          if (e || !tail->fwd_nats) continue;
          // Forward stage on this profile's Viterbi passes (Fig 1)
          if ((e = compact_flags(B[k].vpass, n, db->d_order, B[k].fl, tail->fwd_ids + ro, tail->n_fwd + i, B[k].tmp,
                                 sk)))
            break;
          s = run_fwd(pi, db, B[k].fl, tail->n_fwd + i, sk, tail->fwd_nats + ro, tail->flags + ro, *SS[k]);
        }
        for (auto* x : SS) delete x;                 // stream-ordered frees on each side stream
        if (s != HMG_OK) return s;
        if (e) return cuda_status(e);
      }
      if (ns > 1) {
        for (int k = 0; k < ns; ++k) {
          if ((e = cudaEventRecord(join[k], side[k]))) return cuda_status(e);
          if ((e = cudaStreamWaitEvent(st, join[k], 0))) return cuda_status(e);
          cudaEventDestroy(join[k]);
        }
        cudaEventDestroy(fork);
      }
      mark(5, st);
    }
  }
  if (e == cudaSuccess) e = cudaGetLastError();
  return cuda_status(e);
}

hmg_status hmg_msv_batch(const hmg_profile* const* profs, int nprof, const hmg_db* db, double F1, void* stream,
                         uint8_t* raw, uint8_t* pass) {
  return msv_batch_impl(profs, nprof, db, F1, stream, raw, pass, nullptr);
}

hmg_status hmg_pipeline_batch(const hmg_profile* const* profs, int nprof, const hmg_db* db, double F1, double F2,
                              void* stream, uint8_t* msv_raw, int16_t* vit_raw, uint8_t* flags,
                              int32_t* survivor_ids, int64_t* n_survivors, float* fwd_nats, int32_t* fwd_ids,
                              int64_t* n_fwd) {
  if (!(F2 > 0.0 && F2 <= 1.0)) return HMG_EINVAL;
  if (db && db->nseq && (!vit_raw || !flags || !survivor_ids || !n_survivors)) return HMG_EINVAL;
  if (db && !db->nseq && !n_survivors) return HMG_EINVAL;
  if ((fwd_nats != nullptr) != (n_fwd != nullptr) || (fwd_nats != nullptr) != (fwd_ids != nullptr))
    return HMG_EINVAL;
  BatchTail t{F2, vit_raw, flags, survivor_ids, n_survivors, fwd_nats, fwd_ids, n_fwd};
  return msv_batch_impl(profs, nprof, db, F1, stream, msv_raw, nullptr, &t);
}

}  // extern "C"
