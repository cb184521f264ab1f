// flb_core.cuh — host-side runtime shared by the C ABI (flb_api.cu) and the per-frame kernel
// instantiation units (flb_inst.cu): key structs, error state, launch configuration and the
// run_* launchers.  Every run_<op><X, T> is explicitly instantiated in exactly one flb_inst.cu
// object (one object per (X, T) frame split, compiled in parallel); flb_api.cu sees only the
// extern declarations at the bottom of this file.
#pragma once
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <map>
#include <memory>
#include <mutex>
#include <string>
#include <vector>

#include "../../include/flb_paillier.h"
#include "flb_kernels.cuh"
#include "flb_tc.cuh"
#include "host_bn.hpp"

using flb::host::Limbs;
namespace H = flb::host;

namespace flb_rt {

inline thread_local std::string g_err;

inline int fail(int code, const std::string& msg) {
  g_err = msg;
  return code;
}

#define FLB_CK(call)                                                                    \
  do {                                                                                  \
    cudaError_t e_ = (call);                                                            \
    if (e_ != cudaSuccess) return fail(FLB_ECUDA, std::string(#call) + ": " + cudaGetErrorString(e_)); \
  } while (0)

constexpr int kBlock = 32;  // one warp per block: occupancy follows the register count exactly
constexpr int kReduceChunk = 64;  // inputs per group in one reduction level

// ----------------------------------------------------------------------------- constant blobs
// All device constants of a key live in one buffer; Blob records word offsets.
struct Blob {
  std::vector<uint32_t> words;
  size_t put(const Limbs& v, size_t w) {
    // 16-byte align every array (uint4 loads)
    while (words.size() % 4) words.push_back(0);
    const size_t off = words.size();
    Limbs r = H::resized(v, w);
    words.insert(words.end(), r.begin(), r.end());
    return off;
  }
  size_t put_raw(const std::vector<uint32_t>& v) {
    while (words.size() % 4) words.push_back(0);
    const size_t off = words.size();
    words.insert(words.end(), v.begin(), v.end());
    return off;
  }
};

struct DevBlob {
  std::mutex mu;
  std::map<int, uint32_t*> per_dev;
  ~DevBlob() {
    for (auto& kv : per_dev) {
      int cur;
      if (cudaGetDevice(&cur) == cudaSuccess) {
        cudaSetDevice(kv.first);
        cudaFree(kv.second);
        cudaSetDevice(cur);
      }
    }
  }
  // device copy of `b` on the current device (uploaded once)
  int get(const Blob& b, uint32_t** out) {
    int dev;
    FLB_CK(cudaGetDevice(&dev));
    std::lock_guard<std::mutex> lk(mu);
    auto it = per_dev.find(dev);
    if (it != per_dev.end()) { *out = it->second; return FLB_OK; }
    uint32_t* p = nullptr;
    FLB_CK(cudaMalloc(&p, b.words.size() * 4));
    FLB_CK(cudaMemcpy(p, b.words.data(), b.words.size() * 4, cudaMemcpyHostToDevice));
    per_dev[dev] = p;
    *out = p;
    return FLB_OK;
  }
};

inline int frame_for_bits(size_t nbits) {
  if (nbits <= 1024) return 1024;
  if (nbits <= 2048) return 2048;
  if (nbits <= 3072) return 3072;
  if (nbits <= 4096) return 4096;
  return 0;
}

}  // namespace flb_rt

using namespace flb_rt;

// ----------------------------------------------------------------------------- key structs
struct flb_pub {
  uint32_t nbits = 0, frame = 0, s = 0, sp = 0;
  Limbs n, n2;
  uint32_t n2_n0inv = 0;
  H::Schedule enc;
  Blob blob;
  size_t o_n2 = 0, o_n = 0, o_R2 = 0, o_R1 = 0, o_nR = 0, o_RL = 0, o_sched = 0;
  // tensor-core Montgomery operands for n^2 (flb_tc.cuh; ct_words in {64, 128}), and the integer 1
  bool tc = false;
  size_t o_tcE1 = 0, o_tcE2 = 0, o_one = 0;
  DevBlob dev;
};

struct flb_priv {
  flb_pub* pub = nullptr;  // owned copy of the public half (for n / frame)
  Limbs p, q;
  struct Prime {
    Limbs P, P2;
    uint32_t P_n0inv, P2_n0inv;
    H::Schedule sched;
    size_t o_P, o_P2, o_R2, o_R3, o_Pinv, o_hR, o_sched;
    size_t o_nR;  // n R mod P^2 (key-holder encryption)
    // tensor-core Montgomery operands for P^2 (flb_tc.cuh): extended Toeplitz K-slices of N', N
    size_t o_tcE1 = 0, o_tcE2 = 0;
  } pr[2];
  bool tc = false;       // P^2 tensor-core operands present (sp in {32, 64, 96, 128})
  bool tc_half = false;  // half-frame P tensor-core operands present (H in {32, 64})
  size_t o_one = 0;      // the integer 1
  size_t o_n = 0, o_qR_n = 0, o_qinvR_p = 0;
  size_t o_q2invR = 0, o_enc_sched = 0;  // key-holder encryption: (q^2)^-1 R mod p^2, schedule of n
  // key-holder encryption v2 (r^n mod P^2 = (r^Q mod P)^P mod P^2): half-frame moduli and schedules
  uint32_t H = 0;                         // half-frame limbs (0: v2 not used for this key size)
  struct Half {
    uint32_t n0inv;
    size_t o_P, o_R2, o_R3;
    size_t o_tcE1 = 0, o_tcE2 = 0;  // tensor-core operands of P in the H frame
  } half[2];
  H::Schedule sched_p, sched_q;           // exponents p and q
  size_t o_sched_p = 0, o_sched_q = 0;
  uint32_t n_n0inv = 0;
  Blob blob;
  DevBlob dev;
  ~flb_priv() { delete pub; }
};

// A generic odd modulus for Table I's mod_mul / mod_pow and RSA (L247–L251): the
// Montgomery constants live in an flb_pub "core" whose n2 slot holds the modulus, so the hom-add and
// scalar-mul kernels serve mod_mul and per-element mod_pow unchanged.
struct flb_mod {
  flb_pub core;
  std::mutex mu;
  struct Sched {
    H::Schedule s;
    std::map<int, uint32_t*> dev;
  };
  std::map<std::vector<uint32_t>, Sched> scheds;  // batch-shared exponents seen so far
  ~flb_mod() {
    int cur;
    if (cudaGetDevice(&cur) != cudaSuccess) return;
    for (auto& kv : scheds)
      for (auto& d : kv.second.dev) {
        cudaSetDevice(d.first);
        cudaFree(d.second);
      }
    cudaSetDevice(cur);
  }
};
namespace flb_rt {

// ----------------------------------------------------------------------------- launching
struct Pool {
  static int prepare() {
    static std::mutex mu;
    static std::map<int, bool> done;
    int dev;
    FLB_CK(cudaGetDevice(&dev));
    std::lock_guard<std::mutex> lk(mu);
    if (!done[dev]) {
      cudaMemPool_t pool;
      FLB_CK(cudaDeviceGetDefaultMemPool(&pool, dev));
      uint64_t thr = ~0ull;
      FLB_CK(cudaMemPoolSetAttribute(pool, cudaMemPoolAttrReleaseThreshold, &thr));
      done[dev] = true;
    }
    return FLB_OK;
  }
};

template <typename K>
inline int resident_blocks(K kernel, int* blocks) {
  static std::mutex mu;
  static std::map<std::pair<int, const void*>, int> cache;
  int dev;
  FLB_CK(cudaGetDevice(&dev));
  std::lock_guard<std::mutex> lk(mu);
  auto key = std::make_pair(dev, (const void*)kernel);
  auto it = cache.find(key);
  if (it != cache.end()) { *blocks = it->second; return FLB_OK; }
  int per_sm = 0, sms = 0;
  FLB_CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kernel, kBlock, 0));
  FLB_CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev));
  if (per_sm < 1) per_sm = 1;
  cache[key] = per_sm * sms;
  *blocks = per_sm * sms;
  return FLB_OK;
}

// Grid for `items` work units of T lanes each: at most the resident capacity (the persistent loop
// takes the rest; balancing the rounds was measured slower on B200).

template <int T, typename K>
inline int grid_for(K kernel, uint64_t items, int* grid) {
  int cap;
  int rc = resident_blocks(kernel, &cap);
  if (rc) return rc;
  const uint64_t per_block = kBlock / T;  // work units per block
  const uint64_t cap_items = (uint64_t)cap * per_block;
  const uint64_t want = std::min(items, cap_items);
  *grid = (int)std::max<uint64_t>(1, (want + per_block - 1) / per_block);
  return FLB_OK;
}

struct Scratch {
  void* p = nullptr;
  cudaStream_t st = nullptr;
  ~Scratch() {
    if (p) cudaFreeAsync(p, st);
  }
  int alloc(size_t bytes, cudaStream_t s) {
    st = s;
    if (bytes == 0) return FLB_OK;
    int rc = Pool::prepare();
    if (rc) return rc;
    FLB_CK(cudaMallocAsync(&p, bytes, s));
    return FLB_OK;
  }
};

#define FLB_LAUNCH_CHECK() FLB_CK(cudaGetLastError())

// ---- encrypt
template <int X, int T>
int run_encrypt(const flb_pub* K, const uint32_t* dev, const uint32_t* m, const uint32_t* r, uint64_t seed,
                uint64_t ctr0, uint32_t* c, size_t count, cudaStream_t st) {
  int grid;
  int rc = grid_for<T>(flb::k_encrypt<X, T>, count, &grid);
  if (rc) return rc;
  const uint64_t G = (uint64_t)grid * kBlock / T;
  Scratch sc;
  rc = sc.alloc((size_t)K->enc.table * G * K->s * 4, st);
  if (rc) return rc;
  flb::EncArgs A;
  A.N2 = {dev + K->o_n2, K->n2_n0inv};
  A.R2 = dev + K->o_R2;
  A.nR = dev + K->o_nR;
  A.sched = dev + K->o_sched;
  A.sched_len = (int)K->enc.ops.size();
  A.table = K->enc.table;
  A.nbits = K->nbits;
  A.pt_words = K->sp;
  A.m = m;
  A.r = r;
  A.c = c;
  A.count = count;
  A.seed = seed;
  A.ctr0 = ctr0;
  A.scratch = (uint32_t*)sc.p;
  flb::k_encrypt<X, T><<<grid, kBlock, 0, st>>>(A);
  FLB_LAUNCH_CHECK();
  return FLB_OK;
}

template <int X, int T>
int run_decrypt(const flb_priv* V, const uint32_t* dev, const uint32_t* c, uint32_t* m, size_t count, cudaStream_t st) {
  int grid;
  int rc = grid_for<T>(flb::k_decrypt<X, T>, count, &grid);
  if (rc) return rc;
  const uint64_t G = (uint64_t)grid * kBlock / T;
  const int table = std::max(V->pr[0].sched.table, V->pr[1].sched.table);
  Scratch sc;
  rc = sc.alloc((size_t)table * G * V->pub->sp * 4, st);
  if (rc) return rc;
  flb::DecArgs A;
  for (int i = 0; i < 2; i++) {
    const auto& R = V->pr[i];
    A.pr[i].P2 = {dev + R.o_P2, R.P2_n0inv};
    A.pr[i].R2 = dev + R.o_R2;
    A.pr[i].R3 = dev + R.o_R3;
    A.pr[i].P = {dev + R.o_P, R.P_n0inv};
    A.pr[i].Pinv = dev + R.o_Pinv;
    A.pr[i].hR = dev + R.o_hR;
    A.pr[i].sched = dev + R.o_sched;
    A.pr[i].sched_len = (int)R.sched.ops.size();
    A.pr[i].table = R.sched.table;
  }
  A.n = {dev + V->o_n, V->n_n0inv};
  A.qR_n = dev + V->o_qR_n;
  A.qinvR_p = dev + V->o_qinvR_p;
  A.c = c;
  A.m = m;
  A.count = count;
  A.scratch = (uint32_t*)sc.p;
  flb::k_decrypt<X, T><<<grid, kBlock, 0, st>>>(A);
  FLB_LAUNCH_CHECK();
  return FLB_OK;
}

template <int X, int T>
int run_encrypt_crt(const flb_priv* V, const uint32_t* dev, const uint32_t* m, const uint32_t* r, uint64_t seed,
                    uint64_t ctr0, uint32_t* c, size_t count, cudaStream_t st) {
  int grid;
  int rc = grid_for<T>(flb::k_encrypt_crt<X, T>, count, &grid);
  if (rc) return rc;
  const uint64_t G = (uint64_t)grid * kBlock / T;
  const flb_pub* K = V->pub;
  Scratch sc;
  rc = sc.alloc((size_t)K->enc.table * G * K->sp * 4, st);
  if (rc) return rc;
  flb::EncCrtArgs A;
  for (int i = 0; i < 2; i++) {
    A.P2[i] = {dev + V->pr[i].o_P2, V->pr[i].P2_n0inv};
    A.R2[i] = dev + V->pr[i].o_R2;
    A.nR[i] = dev + V->pr[i].o_nR;
  }
  A.q2 = dev + V->pr[1].o_P2;
  A.q2invR = dev + V->o_q2invR;
  A.sched = dev + V->o_enc_sched;
  A.sched_len = (int)K->enc.ops.size();
  A.table = K->enc.table;
  A.nbits = K->nbits;
  A.m = m;
  A.r = r;
  A.c = c;
  A.count = count;
  A.seed = seed;
  A.ctr0 = ctr0;
  A.scratch = (uint32_t*)sc.p;
  flb::k_encrypt_crt<X, T><<<grid, kBlock, 0, st>>>(A);
  FLB_LAUNCH_CHECK();
  return FLB_OK;
}

template <int X, int T>
int run_modpow(const flb_pub* K, const uint32_t* dev, const uint32_t* sched, const H::Schedule* S, const uint32_t* base,
               uint32_t* out, size_t count, cudaStream_t st) {
  int grid;
  int rc = grid_for<T>(flb::k_modpow<X, T>, count, &grid);
  if (rc) return rc;
  const uint64_t G = (uint64_t)grid * kBlock / T;
  Scratch sc;
  rc = sc.alloc((size_t)S->table * G * K->s * 4, st);
  if (rc) return rc;
  flb::PowArgs A;
  A.N = {dev + K->o_n2, K->n2_n0inv};
  A.R2 = dev + K->o_R2;
  A.sched = sched;
  A.sched_len = (int)S->ops.size();
  A.table = S->table;
  A.base = base;
  A.out = out;
  A.count = count;
  A.scratch = (uint32_t*)sc.p;
  flb::k_modpow<X, T><<<grid, kBlock, 0, st>>>(A);
  FLB_LAUNCH_CHECK();
  return FLB_OK;
}

template <int X, int T>
int run_horner(const flb_pub* K, const uint32_t* dev, const uint32_t* P, uint32_t planes, uint32_t* out, size_t nseg,
               cudaStream_t st) {
  int grid;
  int rc = grid_for<T>(flb::k_horner<X, T>, nseg, &grid);
  if (rc) return rc;
  flb::HornerArgs A;
  A.N2 = {dev + K->o_n2, K->n2_n0inv};
  A.R1 = dev + K->o_R1;
  A.R2 = dev + K->o_R2;
  A.P = P;
  A.K = planes;
  A.out = out;
  A.nseg = nseg;
  flb::k_horner<X, T><<<grid, kBlock, 0, st>>>(A);
  FLB_LAUNCH_CHECK();
  return FLB_OK;
}

template <int X, int T>
int run_mr(const uint32_t* cand, const uint32_t* bases, uint32_t rounds, uint64_t seed, uint64_t ctr0, uint32_t* verdict,
           size_t count, int bw, cudaStream_t st) {
  int grid;
  int rc = grid_for<T>(flb::k_miller_rabin<X, T>, count, &grid);
  if (rc) return rc;
  const uint64_t G = (uint64_t)grid * kBlock / T;
  Scratch sc;
  rc = sc.alloc((size_t)(1u << bw) * G * X * T * 4, st);
  if (rc) return rc;
  flb::MrArgs A;
  A.cand = cand;
  A.bases = bases;
  A.rounds = rounds;
  A.seed = seed;
  A.ctr0 = ctr0;
  A.verdict = verdict;
  A.count = count;
  A.scratch = (uint32_t*)sc.p;
  A.bw = bw;
  flb::k_miller_rabin<X, T><<<grid, kBlock, 0, st>>>(A);
  FLB_LAUNCH_CHECK();
  return FLB_OK;
}

template <int X, int T>
int run_crt_pre(const flb_priv* V, const uint32_t* dev, const uint32_t* r, uint64_t seed, uint64_t ctr0, uint32_t* y,
                size_t count, cudaStream_t st) {
  int grid;
  int rc = grid_for<T>(flb::k_crt_pre<X, T>, count, &grid);
  if (rc) return rc;
  const uint64_t G = (uint64_t)grid * kBlock / T;
  const int table = std::max(V->sched_p.table, V->sched_q.table);
  Scratch sc;
  rc = sc.alloc((size_t)table * G * V->H * 4, st);
  if (rc) return rc;
  flb::CrtPreArgs A;
  for (int i = 0; i < 2; i++) {
    A.P[i] = {dev + V->half[i].o_P, V->half[i].n0inv};
    A.R2[i] = dev + V->half[i].o_R2;
    A.R3[i] = dev + V->half[i].o_R3;
    const H::Schedule& sc_i = i == 0 ? V->sched_q : V->sched_p;  // exponent: the other prime
    A.sched[i] = dev + (i == 0 ? V->o_sched_q : V->o_sched_p);
    A.sched_len[i] = (int)sc_i.ops.size();
    A.table[i] = sc_i.table;
  }
  A.nbits = V->pub->nbits;
  A.pt_words = V->pub->sp;
  A.r = r;
  A.seed = seed;
  A.ctr0 = ctr0;
  A.y = y;
  A.count = count;
  A.scratch = (uint32_t*)sc.p;
  flb::k_crt_pre<X, T><<<grid, kBlock, 0, st>>>(A);
  FLB_LAUNCH_CHECK();
  return FLB_OK;
}

template <int X, int T>
int run_encrypt_crt2(const flb_priv* V, const uint32_t* dev, const uint32_t* m, const uint32_t* y, uint32_t* c,
                     size_t count, cudaStream_t st) {
  int grid;
  int rc = grid_for<T>(flb::k_encrypt_crt2<X, T>, count, &grid);
  if (rc) return rc;
  const uint64_t G = (uint64_t)grid * kBlock / T;
  const int table = std::max(V->sched_p.table, V->sched_q.table);
  Scratch sc;
  rc = sc.alloc((size_t)table * G * V->pub->sp * 4, st);
  if (rc) return rc;
  flb::EncCrt2Args A;
  for (int i = 0; i < 2; i++) {
    A.P2[i] = {dev + V->pr[i].o_P2, V->pr[i].P2_n0inv};
    A.R2[i] = dev + V->pr[i].o_R2;
    A.nR[i] = dev + V->pr[i].o_nR;
    const H::Schedule& sc_i = i == 0 ? V->sched_p : V->sched_q;  // exponent P for P^2
    A.sched[i] = dev + (i == 0 ? V->o_sched_p : V->o_sched_q);
    A.sched_len[i] = (int)sc_i.ops.size();
    A.table[i] = sc_i.table;
  }
  A.q2 = dev + V->pr[1].o_P2;
  A.q2invR = dev + V->o_q2invR;
  A.m = m;
  A.y = y;
  A.H = V->H;
  A.c = c;
  A.count = count;
  A.scratch = (uint32_t*)sc.p;
  flb::k_encrypt_crt2<X, T><<<grid, kBlock, 0, st>>>(A);
  FLB_LAUNCH_CHECK();
  return FLB_OK;
}

// ----------------------------------------------------------------------------- tensor-core modexp
// One k_tc_exp launch over the (up to two) problems of A: persistent grid of two 256-thread CTAs
// per SM (flb_tc.cuh), window-table scratch sized for the largest table.
template <typename F>
int tc_set_attrs(F* kern, int smem_bytes) {
  int dev_id = 0;
  FLB_CK(cudaGetDevice(&dev_id));
  static std::mutex mu;
  static std::map<std::pair<const void*, int>, bool> done;  // function attributes are per device
  std::lock_guard<std::mutex> lk(mu);
  auto key = std::make_pair((const void*)kern, dev_id);
  if (!done[key]) {
    FLB_CK(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, smem_bytes));
    FLB_CK(cudaFuncSetAttribute(kern, cudaFuncAttributePreferredSharedMemoryCarveout, 100));
    done[key] = true;
  }
  return FLB_OK;
}

// tile counts of A's problems; total tiles and the largest window table
inline int tc_tiles(flb::tc::ExpArgs& A, uint64_t* tiles, int* table) {
  *tiles = 0;
  *table = 1;
  for (int i = 0; i < A.nprob; i++) {
    auto& P = A.pb[i];
    if (P.sched_len < 2) return fail(FLB_EUNSUPPORTED, "tensor-core path needs a multi-window exponent");
    P.tiles = (P.count + flb::tc::kTileM - 1) / flb::tc::kTileM;
    *tiles += P.tiles;
    *table = std::max(*table, P.table);
  }
  if (A.nprob < 2) A.pb[1].tiles = 0;
  return FLB_OK;
}

// Half units for a launch's incomplete last round (flb_tc.cuh): on, except while the host pipeline
// runs concurrent chunk launches whose successors fill each other's tails (flb_host_pipeline.cu,
// through flb::set_half_units; per calling thread)
inline thread_local bool tl_half_units = true;

inline int sm_count(int* sms) {
  int dev_id = 0;
  FLB_CK(cudaGetDevice(&dev_id));
  FLB_CK(cudaDeviceGetAttribute(sms, cudaDevAttrMultiProcessorCount, dev_id));
  return FLB_OK;
}

template <int S>
int launch_tc_exp(flb::tc::ExpArgs& A, cudaStream_t st) {
  using C = flb::tc::Cfg<S>;
  int rc = tc_set_attrs(flb::tc::k_tc_exp<S>, C::SMEM);
  if (rc) return rc;
  int sms = 0;
  rc = sm_count(&sms);
  if (rc) return rc;
  uint64_t tiles = 0;
  int table = 1;
  rc = tc_tiles(A, &tiles, &table);
  if (rc) return rc;
  if (tiles == 0) return FLB_OK;
  const int grid = (int)std::min<uint64_t>((uint64_t)(C::CTAS_PER_SM * sms), tiles);
  Scratch s_tab;
  rc = s_tab.alloc((size_t)grid * flb::tc::kTileM * (table + 1) * S * 4, st);
  if (rc) return rc;
  A.scratch = (uint32_t*)s_tab.p;
  A.tab_entries = table + 1;
  A.half_units = tl_half_units ? 1 : 0;
  flb::tc::k_tc_exp<S><<<grid, C::THREADS, C::SMEM, st>>>(A);
  FLB_LAUNCH_CHECK();
  return FLB_OK;
}

// both key-holder stages in one k_tc_exp_dag launch (stage-1 problems A1 at S1 words, stage-2 problems
// A2 at S2 words, the same element counts)
template <int S1, int S2>
int launch_tc_exp_dag(flb::tc::ExpArgs& A1, flb::tc::ExpArgs& A2, cudaStream_t st) {
  constexpr int SMEM = flb::tc::Cfg<S1>::SMEM > flb::tc::Cfg<S2>::SMEM ? flb::tc::Cfg<S1>::SMEM
                                                                       : flb::tc::Cfg<S2>::SMEM;
  int rc = tc_set_attrs(flb::tc::k_tc_exp_dag<S1, S2>, SMEM);
  if (rc) return rc;
  int sms = 0;
  rc = sm_count(&sms);
  if (rc) return rc;
  uint64_t t1 = 0, t2 = 0;
  int tab1 = 1, tab2 = 1;
  rc = tc_tiles(A1, &t1, &tab1);
  if (rc) return rc;
  rc = tc_tiles(A2, &t2, &tab2);
  if (rc) return rc;
  if (A1.nprob != 2 || A2.nprob != 2 || A1.pb[0].tiles != A2.pb[0].tiles || A1.pb[1].tiles != A2.pb[1].tiles)
    return fail(FLB_EINVAL, "dag launch: the two stages must have the same problems' tile counts");
  if (t1 == 0) return FLB_OK;
  if (t1 >= 0xFFFFFFF0ull / 2) return fail(FLB_EINVAL, "dag launch: too many tiles");
  // CTAs per SM (2: one tile's product phase overlaps the other's MMA / normalisation); FLB_TC_CPS=1
  // is a measurement knob (one tile per SM, no overlap)
  static const int cps = [] {
    const char* e = getenv("FLB_TC_CPS");
    return (e && atoi(e) == 1) ? 1 : 2;
  }();
  const int grid = (int)std::min<uint64_t>((uint64_t)(cps * sms), t1 + t2);
  const uint64_t stride = (uint64_t)flb::tc::kTileM * std::max<uint64_t>((uint64_t)(tab1 + 1) * S1,
                                                                          (uint64_t)(tab2 + 1) * S2);
  Scratch s_tab, s_sync;
  rc = s_tab.alloc((size_t)grid * stride * 4, st);
  if (rc) return rc;
  rc = s_sync.alloc((size_t)(1 + t1) * 4, st);
  if (rc) return rc;
  FLB_CK(cudaMemsetAsync(s_sync.p, 0, (size_t)(1 + t1) * 4, st));
  A1.scratch = A2.scratch = (uint32_t*)s_tab.p;
  A1.tab_entries = tab1 + 1;
  A1.half_units = A2.half_units = tl_half_units ? 1 : 0;
  A2.tab_entries = tab2 + 1;
  static_assert(flb::tc::Cfg<S1>::THREADS == flb::tc::Cfg<S2>::THREADS, "one CTA shape for both stages");
  flb::tc::k_tc_exp_dag<S1, S2><<<grid, flb::tc::Cfg<S2>::THREADS, SMEM, st>>>(A1, A2, (uint32_t*)s_sync.p, stride);
  FLB_LAUNCH_CHECK();
  return FLB_OK;
}

// debug: the tensor-core kernel's product phase alone (flb_debug_tc_product)
template <int S>
int run_tc_debug_product(const uint32_t* a, const uint32_t* b, uint32_t* t, uint32_t count, int sq, cudaStream_t st) {
  using C = flb::tc::Cfg<S>;
  // sq: 0 = general product, 1 = block squaring with one triangular diagonal square per lane,
  // 2 = the half-split diagonal square (the form k_tc_exp and stage 1 of k_tc_exp_dag use)
  if (sq == 2) {
    FLB_CK(cudaFuncSetAttribute(flb::tc::k_tc_debug_product<S, 2>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                C::SMEM));
    flb::tc::k_tc_debug_product<S, 2><<<1, C::THREADS, C::SMEM, st>>>(a, b, t, count, 1);
  } else {
    FLB_CK(cudaFuncSetAttribute(flb::tc::k_tc_debug_product<S, 1>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                C::SMEM));
    flb::tc::k_tc_debug_product<S, 1><<<1, C::THREADS, C::SMEM, st>>>(a, b, t, count, sq);
  }
  FLB_LAUNCH_CHECK();
  return FLB_OK;
}

// key-holder stage 2 on the tensor cores: c_P = (1 + m n) y_P^P mod P^2 for both primes in one
// k_tc_exp launch, then k_crt_combine
// stage-2 problems: c_P = (1 + m n) y_P^P mod P^2 for both primes (y = [2][count][H], out cpq [2][count][S])
template <int S>
void tc_stage2_args(const flb_priv* V, const uint32_t* dev, const uint32_t* m, const uint32_t* y, uint32_t* cpq,
                    size_t count, flb::tc::ExpArgs& A) {
  A = flb::tc::ExpArgs{};
  A.nprob = 2;
  A.one = dev + V->o_one;
  for (int i = 0; i < 2; i++) {
    const auto& R = V->pr[i];
    const H::Schedule& sc = i == 0 ? V->sched_p : V->sched_q;  // exponent P for P^2
    auto& P = A.pb[i];
    P.N = dev + R.o_P2;
    P.R2 = dev + R.o_R2;
    P.R3 = dev + R.o_R3;
    P.E1 = dev + R.o_tcE1;
    P.E2 = dev + R.o_tcE2;
    P.sched = dev + (i == 0 ? V->o_sched_p : V->o_sched_q);
    P.sched_len = (int)sc.ops.size();
    P.table = sc.table;
    P.x = y + (size_t)i * count * V->H;
    P.x_stride = V->H;
    P.x_words = V->H;
    P.m = m;
    P.m_stride = P.m_words = V->pub->sp;
    P.nR = dev + R.o_nR;
    P.out = cpq + (size_t)i * count * S;
    P.count = count;
  }
}

// c = CRT(c_p, c_q) for the key-holder encryption (k_crt_combine)
template <int S>
int tc_combine(const flb_priv* V, const uint32_t* dev, const uint32_t* cpq, uint32_t* c, size_t count,
               cudaStream_t st) {
  constexpr int XC = S % 96 == 0 ? 12 : 16, TC = S / XC;  // (S = 96: eight lanes of 12 limbs)
  int cgrid;
  int rc = grid_for<TC>(flb::k_crt_combine<XC, TC>, count, &cgrid);
  if (rc) return rc;
  flb::CombineArgs B;
  B.P2 = {dev + V->pr[0].o_P2, V->pr[0].P2_n0inv};
  B.q2 = dev + V->pr[1].o_P2;
  B.q2invR = dev + V->o_q2invR;
  B.cp = cpq;
  B.cq = cpq + (size_t)count * S;
  B.c = c;
  B.count = count;
  flb::k_crt_combine<XC, TC><<<cgrid, kBlock, 0, st>>>(B);
  FLB_LAUNCH_CHECK();
  return FLB_OK;
}

// key-holder stage 2 on the tensor cores: c_P = (1 + m n) y_P^P mod P^2 for both primes in one
// k_tc_exp launch, then k_crt_combine
template <int S>
int run_encrypt_crt_tc(const flb_priv* V, const uint32_t* dev, const uint32_t* m, const uint32_t* y, uint32_t* c,
                       size_t count, cudaStream_t st) {
  Scratch s_out;
  int rc = s_out.alloc((size_t)2 * count * S * 4, st);
  if (rc) return rc;
  uint32_t* cpq = (uint32_t*)s_out.p;
  flb::tc::ExpArgs A;
  tc_stage2_args<S>(V, dev, m, y, cpq, count, A);
  rc = launch_tc_exp<S>(A, st);
  if (rc) return rc;
  return tc_combine<S>(V, dev, cpq, c, count, st);
}

// r drawn on the device exactly as the CIOS encrypt kernel does (Philox, reading c4): [count][sp]
inline int philox_fill(uint32_t sp, uint32_t nbits, uint64_t seed, uint64_t ctr0, size_t count, Scratch& s_r,
                       cudaStream_t st) {
  int rc = s_r.alloc((size_t)count * sp * 4, st);
  if (rc) return rc;
  int g;
  switch (sp) {
#define FLB_FILL(SPW)                                                                          \
  case SPW:                                                                                    \
    rc = grid_for<4>(flb::k_philox_fill<SPW / 4, 4>, count, &g); /* groups of 4 lanes (T a power of 2) */ \
    if (rc) return rc;                                                                         \
    flb::k_philox_fill<SPW / 4, 4><<<g, kBlock, 0, st>>>((uint32_t*)s_r.p, count, nbits, seed, ctr0); \
    break;
    FLB_FILL(32)
    FLB_FILL(64)
    FLB_FILL(96)
    FLB_FILL(128)
#undef FLB_FILL
    default:
      return fail(FLB_EUNSUPPORTED, "tensor-core path: unsupported plaintext frame");
  }
  FLB_LAUNCH_CHECK();
  return FLB_OK;
}

// public-key encryption on the tensor cores (Eq. 3): c = (1 + m n) r^n mod n^2 in the
// S = ct_words frame, every Montgomery product of the modexp with its reduction as u8 MMAs against
// the Toeplitz operands of n^2 (one problem, k_tc_exp<S>)
// key-holder encryption in one stage on the tensor cores (keys without a half frame, 1024 bits):
// c_P = (1 + m n) r^n mod P^2 for both primes in one k_tc_exp launch (x = r < n < R enters the
// Montgomery domain by one product with R^2), then k_crt_combine; r drawn as k_encrypt_crt does
template <int S>
int run_encrypt_crt1_tc(const flb_priv* V, const uint32_t* dev, const uint32_t* m, const uint32_t* r, uint64_t seed,
                        uint64_t ctr0, uint32_t* c, size_t count, cudaStream_t st) {
  const flb_pub* K = V->pub;
  Scratch s_r, s_out;
  int rc;
  if (!r) {
    rc = philox_fill(K->sp, K->nbits, seed, ctr0, count, s_r, st);
    if (rc) return rc;
    r = (const uint32_t*)s_r.p;
  }
  rc = s_out.alloc((size_t)2 * count * S * 4, st);
  if (rc) return rc;
  uint32_t* cpq = (uint32_t*)s_out.p;
  flb::tc::ExpArgs A{};
  A.nprob = 2;
  A.one = dev + V->o_one;
  for (int i = 0; i < 2; i++) {
    const auto& R = V->pr[i];
    auto& P = A.pb[i];
    P.N = dev + R.o_P2;
    P.R2 = dev + R.o_R2;
    P.R3 = dev + R.o_R3;
    P.E1 = dev + R.o_tcE1;
    P.E2 = dev + R.o_tcE2;
    P.sched = dev + V->o_enc_sched;  // exponent n
    P.sched_len = (int)K->enc.ops.size();
    P.table = K->enc.table;
    P.x = r;
    P.x_stride = P.x_words = K->sp;
    P.m = m;
    P.m_stride = P.m_words = K->sp;
    P.nR = dev + R.o_nR;
    P.out = cpq + (size_t)i * count * S;
    P.count = count;
  }
  rc = launch_tc_exp<S>(A, st);
  if (rc) return rc;
  return tc_combine<S>(V, dev, cpq, c, count, st);
}

template <int S>
int run_encrypt_pub_tc(const flb_pub* K, const uint32_t* dev, const uint32_t* m, const uint32_t* r, uint64_t seed,
                       uint64_t ctr0, uint32_t* c, size_t count, cudaStream_t st) {
  Scratch s_r;
  if (!r) {
    int rc = philox_fill(K->sp, K->nbits, seed, ctr0, count, s_r, st);
    if (rc) return rc;
    r = (const uint32_t*)s_r.p;
  }
  flb::tc::ExpArgs A{};
  A.nprob = 1;
  A.one = dev + K->o_one;
  auto& P = A.pb[0];
  P.N = dev + K->o_n2;
  P.R2 = dev + K->o_R2;
  P.R3 = nullptr;
  P.E1 = dev + K->o_tcE1;
  P.E2 = dev + K->o_tcE2;
  P.sched = dev + K->o_sched;
  P.sched_len = (int)K->enc.ops.size();
  P.table = K->enc.table;
  P.x = r;
  P.x_stride = P.x_words = K->sp;
  P.m = m;
  P.m_stride = P.m_words = K->sp;
  P.nR = dev + K->o_nR;
  P.out = c;
  P.count = count;
  return launch_tc_exp<S>(A, st);
}

// key-holder stage 1 on the tensor cores: y_P = r^Q mod P in the H-word frame (both primes, one
// launch); r drawn by k_philox_fill unless the caller passes it
template <int HS>
int tc_stage1_args(const flb_priv* V, const uint32_t* dev, const uint32_t* r, uint64_t seed, uint64_t ctr0,
                   uint32_t* y, size_t count, cudaStream_t st, Scratch& s_r, flb::tc::ExpArgs& A) {
  const uint32_t sp = V->pub->sp;
  if (!r) {
    int rc = philox_fill(sp, V->pub->nbits, seed, ctr0, count, s_r, st);
    if (rc) return rc;
    r = (const uint32_t*)s_r.p;
  }
  A = flb::tc::ExpArgs{};
  A.nprob = 2;
  A.one = dev + V->o_one;
  for (int i = 0; i < 2; i++) {
    const H::Schedule& sc = i == 0 ? V->sched_q : V->sched_p;  // exponent: the other prime
    auto& P = A.pb[i];
    P.N = dev + V->half[i].o_P;
    P.R2 = dev + V->half[i].o_R2;
    P.R3 = dev + V->half[i].o_R3;
    P.E1 = dev + V->half[i].o_tcE1;
    P.E2 = dev + V->half[i].o_tcE2;
    P.sched = dev + (i == 0 ? V->o_sched_q : V->o_sched_p);
    P.sched_len = (int)sc.ops.size();
    P.table = sc.table;
    P.x = r;
    P.x_stride = sp;
    P.x_words = sp;
    P.m = nullptr;
    P.out = y + (size_t)i * count * HS;
    P.count = count;
  }
  return FLB_OK;
}

template <int HS>
int run_crt_pre_tc(const flb_priv* V, const uint32_t* dev, const uint32_t* r, uint64_t seed, uint64_t ctr0,
                   uint32_t* y, size_t count, cudaStream_t st) {
  Scratch s_r;
  flb::tc::ExpArgs A;
  int rc = tc_stage1_args<HS>(V, dev, r, seed, ctr0, y, count, st, s_r, A);
  if (rc) return rc;
  return launch_tc_exp<HS>(A, st);
}

// both key-holder stages in one dependency-ordered launch (k_tc_exp_dag), then k_crt_combine:
// y_P = r^Q mod P (HS words), c_P = (1 + m n) y_P^P mod P^2 (S words), c = CRT(c_p, c_q)
template <int HS, int S>
int run_encrypt_kh_dag(const flb_priv* V, const uint32_t* dev, const uint32_t* m, const uint32_t* r, uint64_t seed,
                       uint64_t ctr0, uint32_t* c, size_t count, cudaStream_t st) {
  Scratch s_r, s_y, s_out;
  int rc = s_y.alloc((size_t)2 * count * HS * 4, st);
  if (rc) return rc;
  rc = s_out.alloc((size_t)2 * count * S * 4, st);
  if (rc) return rc;
  flb::tc::ExpArgs A1, A2;
  rc = tc_stage1_args<HS>(V, dev, r, seed, ctr0, (uint32_t*)s_y.p, count, st, s_r, A1);
  if (rc) return rc;
  tc_stage2_args<S>(V, dev, m, (const uint32_t*)s_y.p, (uint32_t*)s_out.p, count, A2);
  rc = launch_tc_exp_dag<HS, S>(A1, A2, st);
  if (rc) return rc;
  return tc_combine<S>(V, dev, (const uint32_t*)s_out.p, c, count, st);
}

// decryption with both exponentiations c^(P-1) mod P^2 on the tensor cores (one launch), then the
// CRT tail k_dec_finish on the CUDA cores
template <int S>
int run_decrypt_tc(const flb_priv* V, const uint32_t* dev, const uint32_t* c, uint32_t* m, size_t count,
                   cudaStream_t st) {
  Scratch s_x;
  int rc = s_x.alloc((size_t)2 * count * S * 4, st);
  if (rc) return rc;
  uint32_t* xp = (uint32_t*)s_x.p;
  flb::tc::ExpArgs A{};
  A.nprob = 2;
  A.one = dev + V->o_one;
  for (int i = 0; i < 2; i++) {
    const auto& R = V->pr[i];
    auto& P = A.pb[i];
    P.N = dev + R.o_P2;
    P.R2 = dev + R.o_R2;
    P.R3 = dev + R.o_R3;
    P.E1 = dev + R.o_tcE1;
    P.E2 = dev + R.o_tcE2;
    P.sched = dev + R.o_sched;  // exponent P - 1
    P.sched_len = (int)R.sched.ops.size();
    P.table = R.sched.table;
    P.x = c;
    P.x_stride = 2 * S;
    P.x_words = 2 * S;
    P.m = nullptr;
    P.out = xp + (size_t)i * count * S;
    P.count = count;
  }
  rc = launch_tc_exp<S>(A, st);
  if (rc) return rc;
  constexpr int XF = S % 96 == 0 ? 12 : 16, TF = S / XF;
  int grid;
  rc = grid_for<TF>(flb::k_dec_finish<XF, TF>, count, &grid);
  if (rc) return rc;
  flb::DecArgs D{};
  for (int i = 0; i < 2; i++) {
    const auto& R = V->pr[i];
    D.pr[i].P = {dev + R.o_P, R.P_n0inv};
    D.pr[i].Pinv = dev + R.o_Pinv;
    D.pr[i].hR = dev + R.o_hR;
  }
  D.n = {dev + V->o_n, V->n_n0inv};
  D.qR_n = dev + V->o_qR_n;
  D.qinvR_p = dev + V->o_qinvR_p;
  D.xp = xp;
  D.m = m;
  D.count = count;
  flb::k_dec_finish<XF, TF><<<grid, kBlock, 0, st>>>(D);
  FLB_LAUNCH_CHECK();
  return FLB_OK;
}

template <int X, int T, bool DEBUG>
int run_add(const flb_pub* K, const uint32_t* dev, const uint32_t* a, const uint32_t* b, uint32_t* out, size_t count,
            cudaStream_t st) {
  auto kern = DEBUG ? flb::k_mont<X, T> : flb::k_add<X, T>;
  int grid;
  int rc = grid_for<T>(kern, count, &grid);
  if (rc) return rc;
  flb::AddArgs A;
  A.N2 = {dev + K->o_n2, K->n2_n0inv};
  A.R2 = dev + K->o_R2;
  A.c1 = a;
  A.c2 = b;
  A.out = out;
  A.count = count;
  kern<<<grid, kBlock, 0, st>>>(A);
  FLB_LAUNCH_CHECK();
  return FLB_OK;
}

template <int X, int T>
int run_smul(const flb_pub* K, const uint32_t* dev, const uint32_t* c, const uint32_t* e, uint32_t e_words,
             uint32_t* out, size_t count, cudaStream_t st) {
  int grid;
  int rc = grid_for<T>(flb::k_scalar_mul<X, T>, count, &grid);
  if (rc) return rc;
  const uint64_t G = (uint64_t)grid * kBlock / T;
  const uint32_t ebits = 32 * e_words;
  const int bw = ebits <= 64 ? 3 : (ebits <= 512 ? 5 : 6);
  Scratch sc;
  rc = sc.alloc((size_t)(1u << bw) * G * K->s * 4, st);
  if (rc) return rc;
  flb::SmulArgs A;
  A.N2 = {dev + K->o_n2, K->n2_n0inv};
  A.R2 = dev + K->o_R2;
  A.R1 = dev + K->o_R1;
  A.c = c;
  A.e = e;
  A.e_words = e_words;
  A.bw = bw;
  A.out = out;
  A.count = count;
  A.scratch = (uint32_t*)sc.p;
  flb::k_scalar_mul<X, T><<<grid, kBlock, 0, st>>>(A);
  FLB_LAUNCH_CHECK();
  return FLB_OK;
}

template <int X, int T>
int run_reduce(const flb_pub* K, const uint32_t* dev, const uint32_t* c, size_t num_entries, const int64_t* idx,
               const int64_t* offsets, size_t nseg, size_t max_len, uint32_t* out, cudaStream_t st) {
  const int C = kReduceChunk;
  const size_t num_inputs = num_entries;  // chunk bounds follow the entries (idx may repeat inputs)
  if (max_len == 0 || max_len > num_entries) max_len = std::max<size_t>(num_entries, 1);
  int levels = 1;
  for (size_t cap = C; cap < max_len; cap *= C) levels++;
  // per-level buffers: chunk offsets [nseg+1], starts/ends [max_chunks], partials
  const size_t max_chunks0 = num_inputs / C + nseg + 1;
  Scratch s_plan, s_part0, s_part1;
  const size_t plan_words = (nseg + 1) + 2 * max_chunks0;
  int rc = s_plan.alloc(plan_words * sizeof(int64_t), st);
  if (rc) return rc;
  int64_t* chunk_off = (int64_t*)s_plan.p;
  int64_t* cstart = chunk_off + (nseg + 1);
  int64_t* cend = cstart + max_chunks0;
  // partial buffers (ping-pong), sized for level 0 output
  if (levels > 1) {
    rc = s_part0.alloc(max_chunks0 * K->s * 4, st);
    if (rc) return rc;
    if (levels > 2) {
      rc = s_part1.alloc((max_chunks0 / C + nseg + 1) * K->s * 4, st);
      if (rc) return rc;
    }
  }
  int grid_r;
  rc = grid_for<T>(flb::k_reduce<X, T>, max_chunks0, &grid_r);
  if (rc) return rc;
  const uint32_t* in = c;
  const int64_t* cur_idx = idx;
  const int64_t* cur_off = offsets;
  // level-(>0) offsets must survive while the next plan is built: keep two offset arrays
  Scratch s_off;
  rc = s_off.alloc(2 * (nseg + 1) * sizeof(int64_t), st);
  if (rc) return rc;
  int64_t* offbuf[2] = {(int64_t*)s_off.p, (int64_t*)s_off.p + (nseg + 1)};
  size_t in_chunks = max_chunks0;
  for (int lv = 0; lv < levels; lv++) {
    flb::k_plan_scan<<<1, 1024, 0, st>>>(cur_off, (int64_t)nseg, C, chunk_off);
    FLB_LAUNCH_CHECK();
    const int fill_grid = (int)std::min<size_t>(4096, (in_chunks + 255) / 256 + 1);
    flb::k_plan_fill<<<fill_grid, 256, 0, st>>>(cur_off, chunk_off, (int64_t)nseg, C, cstart, cend);
    FLB_LAUNCH_CHECK();
    const bool last = lv == levels - 1;
    uint32_t* dst = last ? out : (uint32_t*)((lv % 2 == 0) ? s_part0.p : s_part1.p);
    flb::RedArgs A;
    A.N2 = {dev + K->o_n2, K->n2_n0inv};
    A.R1 = dev + K->o_R1;
    A.RL = dev + K->o_RL;
    A.in = in;
    A.idx = cur_idx;
    A.cstart = cstart;
    A.cend = cend;
    A.nchunks = chunk_off + nseg;
    A.out = dst;
    A.max_chunks = in_chunks;
    flb::k_reduce<X, T><<<grid_r, kBlock, 0, st>>>(A);
    FLB_LAUNCH_CHECK();
    if (!last) {
      // next level: segments over this level's chunk partials
      int64_t* nxt = offbuf[lv % 2];
      FLB_CK(cudaMemcpyAsync(nxt, chunk_off, (nseg + 1) * sizeof(int64_t), cudaMemcpyDeviceToDevice, st));
      cur_off = nxt;
      in = dst;
      cur_idx = nullptr;
      in_chunks = in_chunks / C + nseg + 1;
    }
  }
  return FLB_OK;
}

}  // namespace flb_rt

// ----------------------------------------------------------------------------- instantiation lists
// (X, T) splits used by the dispatch macros of flb_api.cu: ENC frames run the public-key / generic
// kernels, DEC frames the private-key kernels (sp-limb frames).
#define FLB_ENC_COMBOS(M) M(16, 2) M(16, 4) M(8, 8) M(12, 8) M(16, 8) M(8, 16) M(12, 16) M(16, 16) M(8, 32)
#define FLB_DEC_COMBOS(M) M(16, 2) M(8, 4) M(16, 4) M(8, 8) M(12, 8) M(16, 8) M(8, 16)

#define FLB_ENC_DECLS(EXT, X, T)                                                                                  \
  EXT template int flb_rt::run_encrypt<X, T>(const flb_pub*, const uint32_t*, const uint32_t*, const uint32_t*,  \
                                             uint64_t, uint64_t, uint32_t*, size_t, cudaStream_t);                \
  EXT template int flb_rt::run_modpow<X, T>(const flb_pub*, const uint32_t*, const uint32_t*,                     \
                                            const flb::host::Schedule*, const uint32_t*, uint32_t*, size_t,       \
                                            cudaStream_t);                                                        \
  EXT template int flb_rt::run_horner<X, T>(const flb_pub*, const uint32_t*, const uint32_t*, uint32_t, uint32_t*, \
                                            size_t, cudaStream_t);                                                \
  EXT template int flb_rt::run_mr<X, T>(const uint32_t*, const uint32_t*, uint32_t, uint64_t, uint64_t, uint32_t*, \
                                        size_t, int, cudaStream_t);                                               \
  EXT template int flb_rt::run_crt_pre<X, T>(const flb_priv*, const uint32_t*, const uint32_t*, uint64_t, uint64_t, \
                                             uint32_t*, size_t, cudaStream_t);                                    \
  EXT template int flb_rt::run_add<X, T, false>(const flb_pub*, const uint32_t*, const uint32_t*, const uint32_t*, \
                                                uint32_t*, size_t, cudaStream_t);                                 \
  EXT template int flb_rt::run_add<X, T, true>(const flb_pub*, const uint32_t*, const uint32_t*, const uint32_t*,  \
                                               uint32_t*, size_t, cudaStream_t);                                  \
  EXT template int flb_rt::run_smul<X, T>(const flb_pub*, const uint32_t*, const uint32_t*, const uint32_t*,      \
                                          uint32_t, uint32_t*, size_t, cudaStream_t);                             \
  EXT template int flb_rt::run_reduce<X, T>(const flb_pub*, const uint32_t*, const uint32_t*, size_t,              \
                                            const int64_t*, const int64_t*, size_t, size_t, uint32_t*,            \
                                            cudaStream_t);
#define FLB_DEC_DECLS(EXT, X, T)                                                                                  \
  EXT template int flb_rt::run_decrypt<X, T>(const flb_priv*, const uint32_t*, const uint32_t*, uint32_t*, size_t, \
                                             cudaStream_t);                                                       \
  EXT template int flb_rt::run_encrypt_crt<X, T>(const flb_priv*, const uint32_t*, const uint32_t*,              \
                                                 const uint32_t*, uint64_t, uint64_t, uint32_t*, size_t,          \
                                                 cudaStream_t);                                                   \
  EXT template int flb_rt::run_encrypt_crt2<X, T>(const flb_priv*, const uint32_t*, const uint32_t*,             \
                                                  const uint32_t*, uint32_t*, size_t, cudaStream_t);
#define FLB_TC_DECLS(EXT, S)                                                                                      \
  EXT template int flb_rt::run_encrypt_crt1_tc<S>(const flb_priv*, const uint32_t*, const uint32_t*,             \
                                                  const uint32_t*, uint64_t, uint64_t, uint32_t*, size_t,        \
                                                  cudaStream_t);                                                  \
  EXT template int flb_rt::run_encrypt_crt_tc<S>(const flb_priv*, const uint32_t*, const uint32_t*,              \
                                                 const uint32_t*, uint32_t*, size_t, cudaStream_t);              \
  EXT template int flb_rt::run_crt_pre_tc<S>(const flb_priv*, const uint32_t*, const uint32_t*, uint64_t,        \
                                             uint64_t, uint32_t*, size_t, cudaStream_t);                        \
  EXT template int flb_rt::run_decrypt_tc<S>(const flb_priv*, const uint32_t*, const uint32_t*, uint32_t*,       \
                                             size_t, cudaStream_t);                                              \
  EXT template int flb_rt::run_tc_debug_product<S>(const uint32_t*, const uint32_t*, uint32_t*, uint32_t, int,   \
                                                   cudaStream_t);                                                 \
  EXT template int flb_rt::run_encrypt_pub_tc<S>(const flb_pub*, const uint32_t*, const uint32_t*, const uint32_t*, \
                                                 uint64_t, uint64_t, uint32_t*, size_t, cudaStream_t);
#define FLB_TC_DAG_DECLS(EXT)                                                                                      \
  EXT template int flb_rt::run_encrypt_kh_dag<32, 64>(const flb_priv*, const uint32_t*, const uint32_t*,         \
                                                      const uint32_t*, uint64_t, uint64_t, uint32_t*, size_t,     \
                                                      cudaStream_t);

#ifndef FLB_INST_TU
#define FLB_EXTERN_ENC(X, T) FLB_ENC_DECLS(extern, X, T)
#define FLB_EXTERN_DEC(X, T) FLB_DEC_DECLS(extern, X, T)
FLB_ENC_COMBOS(FLB_EXTERN_ENC)
FLB_DEC_COMBOS(FLB_EXTERN_DEC)
FLB_TC_DECLS(extern, 32)
FLB_TC_DECLS(extern, 64)
FLB_TC_DECLS(extern, 96)
FLB_TC_DECLS(extern, 128)
FLB_TC_DAG_DECLS(extern)
#undef FLB_EXTERN_ENC
#undef FLB_EXTERN_DEC
#endif
