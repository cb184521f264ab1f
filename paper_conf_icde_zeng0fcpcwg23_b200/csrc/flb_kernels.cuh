// flb_kernels.cuh — the batched Paillier / codec kernels (layers L1, L2) for sm_100a.
//
// Every kernel is a persistent grid: a fixed number of thread groups (sized from occupancy, see
// flb_api.cu) loops over the batch.  A warp's groups always take the same number of trips, so
// the shuffles/ballots of flb_bn.cuh never see an inactive lane; elements past the end compute
// on zeros and skip their store.  Exponent schedules shared by the batch (n for encryption,
// p-1 and q-1 for decryption) are read warp-uniformly, so control flow never diverges.
#pragma once
#include <cstdint>
#include "flb_bn.cuh"

// Launch bounds: one-warp blocks; the minimum resident blocks per SM caps registers per thread
// (65536 / (32 * MINB)).  Tuned on B200.
#ifndef FLB_MINB_ENC
#define FLB_MINB_ENC 14
#endif
#ifndef FLB_MINB_DEC
#define FLB_MINB_DEC 14
#endif
#ifndef FLB_MINB_MUL
#define FLB_MINB_MUL 1
#endif

namespace flb {

struct ModRef {
  const uint32_t* n;  // modulus limbs in the kernel's frame
  uint32_t n0inv;     // -n^-1 mod 2^32 (reading c6)
};

// -n0^-1 mod 2^32 by Newton iteration (n0 odd)
__device__ __forceinline__ uint32_t host_free_neg_inv32(uint32_t n0) {
  uint32_t x = n0;
#pragma unroll
  for (int i = 0; i < 5; i++) x *= 2u - n0 * x;
  return 0u - x;
}

// ----------------------------------------------------------------------------- group indexing
template <int T>
struct Grid {
  uint32_t gid, G, wg0;
  int k;
  __device__ __forceinline__ Grid() {
    const uint32_t tid = blockIdx.x * blockDim.x + threadIdx.x;
    gid = tid / T;
    G = (gridDim.x * blockDim.x) / T;
    wg0 = (tid & ~31u) / T;
    k = (int)(threadIdx.x & (T - 1));
  }
};

template <int X, int T>
__device__ __forceinline__ void load_mod(uint32_t (&n)[X], const ModRef& M) {
  const int k = (int)(lane_id() & (T - 1));
  load_limbs<X>(n, M.n + k * X);
}

template <int X, int T>
__device__ __forceinline__ void load_const(uint32_t (&r)[X], const uint32_t* p) {
  const int k = (int)(lane_id() & (T - 1));
  load_limbs<X>(r, p + k * X);
}

template <int X, int T>
__device__ __forceinline__ void set_one(uint32_t (&r)[X]) {
  const int k = (int)(lane_id() & (T - 1));
  zero_limbs<X>(r);
  if (k == 0) r[0] = 1;
}

// Load limbs [k*X, k*X+X) of an element with `words` limbs (words may be < X*T: the rest are 0;
// a chunk straddling `words` is read word by word so no lane reads past the element).
template <int X, int T>
__device__ __forceinline__ void load_elem(uint32_t (&r)[X], const uint32_t* base, uint32_t words, bool valid) {
  const int k = (int)(lane_id() & (T - 1));
  const uint32_t w0 = (uint32_t)(k * X);
  if (valid && w0 + X <= words) {
    load_limbs<X>(r, base + w0);
  } else {
#pragma unroll
    for (int j = 0; j < X; j++) r[j] = (valid && w0 + j < words) ? __ldg(base + w0 + j) : 0u;
  }
}

// ----------------------------------------------------------------------------- Philox4x32-10
// Reading c4: r_i = Philox4x32-10(key = seed, ctr = (i lo, i hi, j, 0)), word 4j+t of r.
__device__ __forceinline__ uint4 philox4x32_10(uint4 c, uint2 key) {
#pragma unroll
  for (int r = 0; r < 10; r++) {
    if (r) { key.x += 0x9E3779B9u; key.y += 0xBB67AE85u; }
    const uint32_t hi0 = __umulhi(0xD2511F53u, c.x), lo0 = 0xD2511F53u * c.x;
    const uint32_t hi1 = __umulhi(0xCD9E8D57u, c.z), lo1 = 0xCD9E8D57u * c.z;
    c = make_uint4(hi1 ^ c.y ^ key.x, lo1, hi0 ^ c.w ^ key.y, lo0);
  }
  return c;
}

// r for element `index`: pt_words Philox words, bits >= nbits-1 cleared, 0 -> 1.
template <int X, int T>
__device__ __forceinline__ void philox_r(uint32_t (&r)[X], uint64_t seed, uint64_t index, uint32_t pt_words,
                                         uint32_t nbits, uint32_t woff = 0, bool fix_zero = true) {
  const int k = (int)(lane_id() & (T - 1));
  const uint2 key = make_uint2((uint32_t)seed, (uint32_t)(seed >> 32));
#pragma unroll
  for (int v = 0; v < X / 4; v++) {
    const uint32_t w0 = woff + (uint32_t)(k * X + 4 * v);
    uint4 o = make_uint4(0, 0, 0, 0);
    if (w0 < pt_words) o = philox4x32_10(make_uint4((uint32_t)index, (uint32_t)(index >> 32), w0 / 4, 0), key);
    r[4 * v] = o.x; r[4 * v + 1] = o.y; r[4 * v + 2] = o.z; r[4 * v + 3] = o.w;
  }
  const uint32_t lim = nbits - 1;  // keep bits [0, nbits-1)
#pragma unroll
  for (int j = 0; j < X; j++) {
    const uint32_t w = woff + (uint32_t)(k * X + j);
    if (w >= pt_words || 32u * w >= lim) r[j] = 0;
    else if (32u * (w + 1) > lim) r[j] &= (1u << (lim - 32u * w)) - 1u;
  }
  if (fix_zero) {
    const bool nz = !all_zero<X>(r);
    const uint32_t bal = __ballot_sync(FULL, nz);
    const int base = (T == 32) ? 0 : (int)(lane_id() & ~(uint32_t)(T - 1));
    const uint32_t gm = (T == 32) ? 0xffffffffu : (((1u << T) - 1u) << base);
    if ((bal & gm) == 0 && k == 0) r[0] = 1;
  }
}

// ----------------------------------------------------------------------------- modexp
// Sliding-window Montgomery exponentiation with a batch-shared schedule (host_bn.hpp
// sliding_schedule).  x: base in Montgomery form (clobbered).  The odd-power table lives in
// global scratch: entry i of this group at tab + i*stride + k*X.
template <int X, int T>
__device__ __forceinline__ void modexp_sched(uint32_t (&acc)[X], uint32_t (&x)[X], const uint32_t* __restrict__ sched,
                                             int len, int table, uint32_t* tab, size_t stride,
                                             const uint32_t (&n)[X], uint32_t n0inv) {
  const int k = (int)(lane_id() & (T - 1));
  uint32_t b[X];
  store_limbs<X>(tab + k * X, x);
  if (table > 1) {
    mont_sqr<X, T>(b, x, n, n0inv);
#pragma unroll 1
    for (int i = 1; i < table; i++) {
      mont_mul<X, T>(x, x, b, n, n0inv);
      store_limbs<X>(tab + (size_t)i * stride + k * X, x);
    }
  }
  const uint32_t op0 = __ldg(sched);
  load_limbs_plain<X>(acc, tab + (size_t)((op0 >> 16) - 1) * stride + k * X);
#pragma unroll 1
  for (int o = 1; o < len; o++) {
    const uint32_t op = __ldg(sched + o);
    const int sq = (int)(op & 0xffffu), idx = (int)(op >> 16) - 1;
    const int steps = sq + (idx >= 0 ? 1 : 0);
#pragma unroll 1
    for (int i = 0; i < steps; i++) {
      if (i == sq) {
        load_limbs_plain<X>(b, tab + (size_t)idx * stride + k * X);
        mont_mul<X, T>(acc, acc, b, n, n0inv);
      } else {
        mont_sqr<X, T>(acc, acc, n, n0inv);
      }
    }
  }
}

// ----------------------------------------------------------------------------- encrypt
struct EncArgs {
  ModRef N2;               // n^2 in the s-limb frame
  const uint32_t* R2;      // R^2 mod n^2
  const uint32_t* nR;      // n*R mod n^2
  const uint32_t* sched;   // schedule of the exponent n
  int sched_len, table;
  uint32_t nbits, pt_words;
  const uint32_t* m;       // [count][pt_words]
  const uint32_t* r;       // [count][pt_words] or null (Philox)
  uint32_t* c;             // [count][2*pt_words]
  uint64_t count, seed, ctr0;
  uint32_t* scratch;       // table * G * S words
};

// c = (1 + m n) r^n mod n^2 (Eq. 3 with g = n+1: g^m = 1 + m n mod n^2).
template <int X, int T>
__global__ void __launch_bounds__(32, FLB_MINB_ENC) k_encrypt(const EncArgs A) {
  constexpr int S = X * T;
  const Grid<T> g;
  uint32_t n[X];
  load_mod<X, T>(n, A.N2);
  const uint32_t n0inv = A.N2.n0inv;
  uint32_t* tab = A.scratch + (size_t)g.gid * S;
  const size_t stride = (size_t)g.G * S;
  for (uint64_t base = g.wg0; base < A.count; base += g.G) {
    const uint64_t e = base + (g.gid - g.wg0);
    const bool valid = e < A.count;
    uint32_t x[X], b[X], acc[X];
    if (A.r) load_elem<X, T>(x, A.r + e * A.pt_words, A.pt_words, valid);
    else philox_r<X, T>(x, A.seed, A.ctr0 + e, A.pt_words, A.nbits);
    load_const<X, T>(b, A.R2);
    mont_mul<X, T>(x, x, b, n, n0inv);                       // r~ = r R mod n^2
    modexp_sched<X, T>(acc, x, A.sched, A.sched_len, A.table, tab, stride, n, n0inv);  // r^n R
    load_elem<X, T>(x, A.m + e * A.pt_words, A.pt_words, valid);
    load_const<X, T>(b, A.nR);
    mont_mul<X, T>(x, x, b, n, n0inv);                       // m n (< n^2, exact)
    grp_add_small<X, T>(x, 1u);                              // 1 + m n
    mont_mul<X, T>(acc, acc, x, n, n0inv);                   // r^n (1 + m n)
    if (valid) store_limbs<X>(A.c + e * S + g.k * X, acc);
  }
}

// ----------------------------------------------------------------------------- decrypt (CRT)
struct PrimeArgs {
  ModRef P2;              // P^2 in the sp frame
  const uint32_t* R2;     // R^2 mod P^2
  const uint32_t* R3;     // R^3 mod P^2
  ModRef P;               // P in the sp frame
  const uint32_t* Pinv;   // P^-1 mod 2^(32 sp)
  const uint32_t* hR;     // h_P R mod P, h_p = (-q)^-1 mod p, h_q = (-p)^-1 mod q
  const uint32_t* sched;  // schedule of P-1
  int sched_len, table;
};
struct DecArgs {
  PrimeArgs pr[2];        // [0] = p (the larger prime), [1] = q
  ModRef n;               // n in the sp frame
  const uint32_t* qR_n;   // q R mod n
  const uint32_t* qinvR_p;// q^-1 R mod p
  const uint32_t* c;      // [count][2 sp]
  uint32_t* m;            // [count][sp]
  uint64_t count;
  uint32_t* scratch;      // max table * G * sp
  const uint32_t* xp;     // k_dec_finish: [2][count][sp], c^(P-1) mod P^2 (canonical)
};

// m = D(c) (Eq. 4) by CRT (reading c10):
//   m_P = L_P(c^(P-1) mod P^2) h_P mod P, m = m_q + q ((m_p - m_q) q^-1 mod p).
template <int X, int T>
__global__ void __launch_bounds__(32, FLB_MINB_DEC) k_decrypt(const DecArgs A) {
  constexpr int S = X * T;  // sp
  const Grid<T> g;
  uint32_t* tab = A.scratch + (size_t)g.gid * S;
  const size_t stride = (size_t)g.G * S;
  for (uint64_t base = g.wg0; base < A.count; base += g.G) {
    const uint64_t e = base + (g.gid - g.wg0);
    const bool valid = e < A.count;
    uint32_t mres[2][X];
#pragma unroll 1
    for (int P = 0; P < 2; P++) {
      const PrimeArgs& pa = A.pr[P];
      uint32_t n[X], lo[X], hi[X], b[X], x[X];
      load_mod<X, T>(n, pa.P2);
      load_elem<X, T>(lo, A.c + e * (2 * S), S, valid);
      load_elem<X, T>(hi, A.c + e * (2 * S) + S, S, valid);
      load_const<X, T>(b, pa.R2);
      mont_mul<X, T>(lo, lo, b, n, pa.P2.n0inv);          // c_lo R mod P^2
      load_const<X, T>(b, pa.R3);
      mont_mul<X, T>(hi, hi, b, n, pa.P2.n0inv);          // c_hi R^2 mod P^2
      const uint32_t cy = grp_add<X, T>(x, lo, hi);
      grp_cond_sub<X, T>(x, n, cy);                       // c R mod P^2 (Montgomery form of c)
      modexp_sched<X, T>(lo, x, pa.sched, pa.sched_len, pa.table, tab, stride, n, pa.P2.n0inv);
      set_one<X, T>(b);
      mont_mul<X, T>(lo, lo, b, n, pa.P2.n0inv);          // c^(P-1) mod P^2
      grp_sub_one<X, T>(lo);                              // x - 1 = L * P
      load_const<X, T>(b, pa.Pinv);
      mul_lo<X, T>(hi, lo, b);                            // L = (x - 1) / P (exact division)
      load_mod<X, T>(n, pa.P);
      load_const<X, T>(b, pa.hR);
      mont_mul<X, T>(x, hi, b, n, pa.P.n0inv);            // m_P = L h_P mod P
#pragma unroll
      for (int j = 0; j < X; j++) {
        if (P == 0) mres[0][j] = x[j];
        else mres[1][j] = x[j];
      }
    }
    uint32_t n[X], d[X], t[X];
    load_mod<X, T>(n, A.pr[0].P);
    const uint32_t br = grp_sub<X, T>(d, mres[0], mres[1]);   // m_p - m_q (m_q < q < p)
#pragma unroll
    for (int j = 0; j < X; j++) t[j] = br ? n[j] : 0u;
    grp_add<X, T>(d, d, t);                                    // mod p
    load_const<X, T>(t, A.qinvR_p);
    mont_mul<X, T>(d, d, t, n, A.pr[0].P.n0inv);               // u = (m_p - m_q) q^-1 mod p
    load_mod<X, T>(n, A.n);
    load_const<X, T>(t, A.qR_n);
    mont_mul<X, T>(d, d, t, n, A.n.n0inv);                     // q u (< n, exact)
    grp_add<X, T>(d, d, mres[1]);                              // m = m_q + q u
    if (valid) store_limbs<X>(A.m + e * S + g.k * X, d);
  }
}

// ----------------------------------------------------------------------------- key-holder encrypt
struct EncCrtArgs {
  ModRef P2[2];            // p^2, q^2 in the sp frame
  const uint32_t* R2[2];   // R^2 mod P^2
  const uint32_t* nR[2];   // n R mod P^2
  const uint32_t* q2;      // q^2 (sp limbs, plain)
  const uint32_t* q2invR;  // (q^2)^-1 R mod p^2
  const uint32_t* sched;   // schedule of the exponent n (same as the public path)
  int sched_len, table;
  uint32_t nbits;
  const uint32_t* m;       // [count][sp]
  const uint32_t* r;       // [count][sp] or null (Philox)
  uint32_t* c;             // [count][2 sp]
  uint64_t count, seed, ctr0;
  uint32_t* scratch;       // table * G * sp
};

// Same bits as k_encrypt (Eq. 3, g = n+1) for a party holding p, q:
//   c_P = (1 + m n) r^n mod P^2 for P in {p, q} (sp-limb moduli, exponent n itself, so every r
//   gives the public-path value), then c = c_q + q^2 ((c_p - c_q) (q^2)^-1 mod p^2) < n^2.
template <int X, int T>
__global__ void __launch_bounds__(32, FLB_MINB_DEC) k_encrypt_crt(const EncCrtArgs A) {
  constexpr int S = X * T;  // sp
  const Grid<T> g;
  uint32_t* tab = A.scratch + (size_t)g.gid * S;
  const size_t stride = (size_t)g.G * S;
  for (uint64_t base = g.wg0; base < A.count; base += g.G) {
    const uint64_t e = base + (g.gid - g.wg0);
    const bool valid = e < A.count;
    uint32_t cres[2][X];
#pragma unroll 1
    for (int P = 0; P < 2; P++) {
      uint32_t n[X], x[X], b[X], acc[X];
      load_mod<X, T>(n, A.P2[P]);
      const uint32_t n0inv = A.P2[P].n0inv;
      if (A.r) load_elem<X, T>(x, A.r + e * S, S, valid);
      else philox_r<X, T>(x, A.seed, A.ctr0 + e, S, A.nbits);
      load_const<X, T>(b, A.R2[P]);
      mont_mul<X, T>(x, x, b, n, n0inv);                       // r R mod P^2
      modexp_sched<X, T>(acc, x, A.sched, A.sched_len, A.table, tab, stride, n, n0inv);  // r^n R
      load_elem<X, T>(x, A.m + e * S, S, valid);
      load_const<X, T>(b, A.nR[P]);
      mont_mul<X, T>(x, x, b, n, n0inv);                       // m n mod P^2
      set_one<X, T>(b);
      const uint32_t cy = grp_add<X, T>(x, x, b);
      grp_cond_sub<X, T>(x, n, cy);                            // 1 + m n mod P^2
      mont_mul<X, T>(acc, acc, x, n, n0inv);                   // c_P
#pragma unroll
      for (int j = 0; j < X; j++) {
        if (P == 0) cres[0][j] = acc[j];
        else cres[1][j] = acc[j];
      }
    }
    uint32_t n[X], d[X], t[X], hi[X];
    load_mod<X, T>(n, A.P2[0]);
    const uint32_t br = grp_sub<X, T>(d, cres[0], cres[1]);   // c_p - c_q (c_q < q^2 < p^2)
#pragma unroll
    for (int j = 0; j < X; j++) t[j] = br ? n[j] : 0u;
    grp_add<X, T>(d, d, t);                                    // mod p^2
    load_const<X, T>(t, A.q2invR);
    mont_mul<X, T>(d, d, t, n, A.P2[0].n0inv);                 // u = (c_p - c_q) q^-2 mod p^2
    load_const<X, T>(t, A.q2);
    mul_full<X, T>(d, hi, d, t);                               // q^2 u (2 sp limbs)
    const uint32_t cy = grp_add<X, T>(d, d, cres[1]);          // + c_q
    grp_add_small<X, T>(hi, cy);
    if (valid) {
      store_limbs<X>(A.c + e * (2 * S) + g.k * X, d);
      store_limbs<X>(A.c + e * (2 * S) + S + g.k * X, hi);
    }
  }
}

// ----------------------------------------------------------------------------- generic mod_pow
struct PowArgs {
  ModRef N;                // any odd modulus in the S-limb frame
  const uint32_t* R2;      // R^2 mod N
  const uint32_t* sched;   // schedule of the batch-shared exponent
  int sched_len, table;
  const uint32_t* base;    // [count][S], each < N
  uint32_t* out;           // [count][S]
  uint64_t count;
  uint32_t* scratch;
};

// out = base^e mod N for one exponent shared by the batch (Table I mod_pow; RSA
// encrypt/decrypt, L248–L249).
template <int X, int T>
__global__ void __launch_bounds__(32, FLB_MINB_ENC) k_modpow(const PowArgs A) {
  constexpr int S = X * T;
  const Grid<T> g;
  uint32_t n[X];
  load_mod<X, T>(n, A.N);
  const uint32_t n0inv = A.N.n0inv;
  uint32_t* tab = A.scratch + (size_t)g.gid * S;
  const size_t stride = (size_t)g.G * S;
  for (uint64_t base = g.wg0; base < A.count; base += g.G) {
    const uint64_t e = base + (g.gid - g.wg0);
    const bool valid = e < A.count;
    uint32_t x[X], b[X], acc[X];
    load_elem<X, T>(x, A.base + e * S, S, valid);
    load_const<X, T>(b, A.R2);
    mont_mul<X, T>(x, x, b, n, n0inv);
    modexp_sched<X, T>(acc, x, A.sched, A.sched_len, A.table, tab, stride, n, n0inv);
    set_one<X, T>(b);
    mont_mul<X, T>(acc, acc, b, n, n0inv);
    if (valid) store_limbs<X>(A.out + e * S + g.k * X, acc);
  }
}

// out[i] = 1 (the empty product / x^0), [count][S]
static __global__ void k_fill_one(uint32_t* out, uint64_t count, uint32_t S) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < count * S; i += (uint64_t)gridDim.x * blockDim.x)
    out[i] = (i % S) == 0 ? 1u : 0u;
}

// ----------------------------------------------------------------------------- FLB_DEBUG_CHECKS
// Value-range checks the hot path does not make (include/flb_paillier.h): each
// counts the offending elements into *bad (one thread per element; debug mode only).
// rows x_i (words limbs, row stride `stride`) with x_i >= bound
static __global__ void k_check_below(const uint32_t* x, uint64_t count, uint32_t stride, const uint32_t* bound,
                                     uint32_t words, unsigned long long* bad) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < count; i += (uint64_t)gridDim.x * blockDim.x) {
    const uint32_t* r = x + i * stride;
    int c = 0;
    for (int w = (int)words - 1; w >= 0 && c == 0; w--) {
      const uint32_t a = r[w], b = __ldg(bound + w);
      c = a < b ? -1 : a > b ? 1 : 0;
    }
    if (c >= 0) atomicAdd(bad, 1ull);
  }
}
// int64 indices outside [0, hi)
static __global__ void k_check_index(const int64_t* idx, uint64_t count, int64_t hi, unsigned long long* bad) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < count; i += (uint64_t)gridDim.x * blockDim.x) {
    const int64_t v = idx[i];
    if (v < 0 || v >= hi) atomicAdd(bad, 1ull);
  }
}
// CSR offsets [segments + 1]: offsets[0] = 0, non-decreasing, offsets[segments] = total
static __global__ void k_check_offsets(const int64_t* off, uint64_t segments, int64_t total, unsigned long long* bad) {
  for (uint64_t j = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; j <= segments; j += (uint64_t)gridDim.x * blockDim.x) {
    const int64_t v = off[j];
    const bool ok = (j == 0 ? v == 0 : v >= off[j - 1]) && (j < segments || v == total);
    if (!ok) atomicAdd(bad, 1ull);
  }
}
// per-plaintext summand counts above the padding capacity 2^pad_bits (b overflow bits)
static __global__ void k_check_counts(const uint32_t* cnt, uint64_t count, uint64_t limit, unsigned long long* bad) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < count; i += (uint64_t)gridDim.x * blockDim.x)
    if ((uint64_t)cnt[i] > limit) atomicAdd(bad, 1ull);
}

// ----------------------------------------------------------------------------- Miller–Rabin (keygen)
struct MrArgs {
  const uint32_t* cand;       // [count][S] odd candidates >= 5
  const uint32_t* bases;      // [count][rounds][S] Montgomery-form bases (< cand), or null: Philox
  uint32_t rounds;
  uint64_t seed, ctr0;
  uint32_t* verdict;          // [count] 1 = passed every round
  uint64_t count;
  uint32_t* scratch;          // 2^bw * G * S
  int bw;
};

// this group's exponent staging (S words): the candidate minus one, read bit-window by bit-window
template <int X, int T>
__device__ __forceinline__ uint32_t* exp_stage_group() {
  constexpr int LD = X + 4;
  __shared__ __align__(16) uint32_t ebuf[kMaxWarps * 32 * LD];
  return ebuf + (threadIdx.x >> 5) * (32 * LD) + (int)(lane_id() & ~(uint32_t)(T - 1)) * LD;
}

template <int X>
__device__ __forceinline__ uint32_t staged_word(const uint32_t* st, int w) {
  return st[(w / X) * (X + 4) + (w % X)];
}

// group-wide equality of two distributed numbers
template <int X, int T>
__device__ __forceinline__ bool grp_equal(const uint32_t (&a)[X], const uint32_t (&b)[X]) {
  uint32_t diff = 0;
#pragma unroll
  for (int j = 0; j < X; j++) diff |= a[j] ^ b[j];
  const uint32_t bal = __ballot_sync(FULL, diff != 0);
  const int base = (T == 32) ? 0 : (int)(lane_id() & ~(uint32_t)(T - 1));
  const uint32_t gm = (T == 32) ? 0xffffffffu : (((1u << T) - 1u) << base);
  return (bal & gm) == 0;
}

// Miller–Rabin rounds for a batch of candidates, each with its own modulus.  Bases
// are taken in Montgomery form (a random a~ < P is the Montgomery form of the random base
// a = a~ R^-1 mod P), so no R^2 mod P is needed; x = a^d is formed by a fixed-window ladder over
// the bits of d = (P-1)/2^s with warp-uniform control (zero digits and not-yet-started lanes
// select instead of branching), then compared with 1 and P-1 after leaving the Montgomery domain.
template <int X, int T>
__global__ void __launch_bounds__(32, FLB_MINB_ENC) k_miller_rabin(const MrArgs A) {
  constexpr int S = X * T;
  const Grid<T> g;
  uint32_t* tab = A.scratch + (size_t)g.gid * S;
  const size_t stride = (size_t)g.G * S;
  const int table = 1 << A.bw;
  uint32_t* est = exp_stage_group<X, T>();
  for (uint64_t base = g.wg0; base < A.count; base += g.G) {
    const uint64_t e = base + (g.gid - g.wg0);
    const bool valid = e < A.count;
    uint32_t n[X], pm1[X], x[X], b[X], acc[X] = {}, y[X], one[X];
    load_elem<X, T>(n, A.cand + e * S, S, valid);
    if (!valid && g.k == 0) n[0] = 5;  // dummy modulus for idle groups
    const uint32_t n0inv = __shfl_sync(FULL, host_free_neg_inv32(n[0]), 0, T);
#pragma unroll
    for (int j = 0; j < X; j++) pm1[j] = n[j];
    if (g.k == 0) pm1[0] &= ~1u;  // P - 1 (P odd)
    set_one<X, T>(one);
    // s = trailing zeros of P - 1; bits(P - 1)
    int lz = -1, hz = -1;
#pragma unroll
    for (int j = X - 1; j >= 0; j--) if (pm1[j]) lz = g.k * X * 32 + j * 32 + (__ffs(pm1[j]) - 1);
#pragma unroll
    for (int j = 0; j < X; j++) if (pm1[j]) hz = g.k * X * 32 + j * 32 + 31 - __clz(pm1[j]);
    int s_bits = lz < 0 ? 0x7fffffff : lz;
#pragma unroll
    for (int o = 1; o < T; o <<= 1) s_bits = min(s_bits, __shfl_xor_sync(FULL, s_bits, o, T));
    int top_bit = hz;
#pragma unroll
    for (int o = 1; o < T; o <<= 1) top_bit = max(top_bit, __shfl_xor_sync(FULL, top_bit, o, T));
    const int dbits = top_bit + 1 - s_bits;  // bits of d
    // stage P - 1 for digit extraction
    __syncwarp();
    {
      uint4* q = reinterpret_cast<uint4*>(est + g.k * (X + 4));
#pragma unroll
      for (int v = 0; v < X / 4; v++) q[v] = make_uint4(pm1[4 * v], pm1[4 * v + 1], pm1[4 * v + 2], pm1[4 * v + 3]);
    }
    __syncwarp();
    int topw = (dbits - 1) / A.bw;
    topw = __reduce_max_sync(FULL, valid ? topw : 0);
    int smax = __reduce_max_sync(FULL, valid ? s_bits : 1);
    bool composite = false;
#pragma unroll 1
    for (uint32_t rd = 0; rd < A.rounds; rd++) {
      if (A.bases) {
        load_elem<X, T>(x, A.bases + (e * A.rounds + rd) * S, S, valid);
      } else {
        philox_r<X, T>(x, A.seed, (A.ctr0 + e) * 64 + rd, S, (uint32_t)(top_bit + 1));
      }
      // table: T[j] = x^j (Montgomery), j = 1 .. table-1
      store_limbs<X>(tab + stride + g.k * X, x);
#pragma unroll
      for (int j = 0; j < X; j++) b[j] = x[j];
#pragma unroll 1
      for (int i = 2; i < table; i++) {
        mont_mul<X, T>(b, b, x, n, n0inv);
        store_limbs<X>(tab + (size_t)i * stride + g.k * X, b);
      }
      bool started = false;
#pragma unroll 1
      for (int w = topw; w >= 0; w--) {
        if (w != topw) {
#pragma unroll 1
          for (int sq = 0; sq < A.bw; sq++) mont_sqr<X, T>(acc, acc, n, n0inv);
        }
        // digit w of d = bits [s + w bw, s + w bw + bw) of P - 1 (zero beyond d's top)
        uint32_t dgt = 0;
        if (w * A.bw < dbits) {
          const int lo = s_bits + w * A.bw, word = lo >> 5, off = lo & 31;
          uint32_t v = staged_word<X>(est, word) >> off;
          if (off + A.bw > 32 && word + 1 < S) v |= staged_word<X>(est, word + 1) << (32 - off);
          const int nb = min(A.bw, dbits - w * A.bw);
          dgt = v & ((1u << nb) - 1u);
        }
        load_limbs_plain<X>(b, tab + (size_t)(dgt ? dgt : 1u) * stride + g.k * X);
        mont_mul<X, T>(y, acc, b, n, n0inv);
#pragma unroll
        for (int j = 0; j < X; j++) acc[j] = dgt ? (started ? y[j] : b[j]) : acc[j];
        started = started || (dgt != 0);
      }
      mont_mul<X, T>(y, acc, one, n, n0inv);  // a^d mod P
      // every lane evaluates every comparison (ballots must never sit in divergent code)
      const bool eq1 = grp_equal<X, T>(y, one), eqm1 = grp_equal<X, T>(y, pm1);
      bool pass = eq1 || eqm1;
#pragma unroll 1
      for (int r = 1; r < smax; r++) {
        mont_sqr<X, T>(acc, acc, n, n0inv);
        mont_mul<X, T>(y, acc, one, n, n0inv);
        const bool eq = grp_equal<X, T>(y, pm1);
        pass = pass || (r < s_bits && eq);
      }
      composite = composite || !pass;
    }
    if (valid && g.k == 0) A.verdict[e] = composite ? 0u : 1u;
  }
}

// candidates for key generation: Philox words, bits above `bits` cleared, top two bits and bit 0
// set (reading c5), limbs above the prime's words zero; one thread per limb.
static __global__ void k_gen_candidates(uint32_t* cand, uint64_t count, uint32_t S, uint32_t bits, uint64_t seed,
                                 uint64_t ctr0) {
  const uint64_t total = count * S;
  for (uint64_t t = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; t < total; t += (uint64_t)gridDim.x * blockDim.x) {
    const uint64_t i = t / S;
    const uint32_t w = (uint32_t)(t - i * S);
    uint32_t v = 0;
    if (32u * w < bits) {
      const uint64_t idx = ctr0 + i;
      const uint4 o = philox4x32_10(make_uint4((uint32_t)idx, (uint32_t)(idx >> 32), w / 4, 0x6b657967u),
                                    make_uint2((uint32_t)seed, (uint32_t)(seed >> 32)));
      v = (&o.x)[w & 3];
      if (32u * (w + 1) > bits) v &= (1u << (bits - 32u * w)) - 1u;
      const uint32_t top = bits - 1;
      if (w == top / 32) v |= 1u << (top % 32);
      if (w == (top - 1) / 32) v |= 1u << ((top - 1) % 32);
      if (w == 0) v |= 1u;
    }
    cand[t] = v;
  }
}

// small-prime sieve: flag[i] = 1 if no prime in `primes` divides candidate i
static __global__ void k_sieve(const uint32_t* __restrict__ cand, uint64_t count, uint32_t S, uint32_t words,
                        const uint32_t* __restrict__ primes, uint32_t nprimes, uint32_t* __restrict__ flag) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < count; i += (uint64_t)gridDim.x * blockDim.x) {
    const uint32_t* c = cand + i * S;
    uint32_t ok = 1;
    for (uint32_t k = 0; k < nprimes && ok; k++) {
      const uint32_t p = __ldg(primes + k);
      uint64_t r = 0;
      for (int w = (int)words - 1; w >= 0; w--) r = ((r << 32) | c[w]) % p;
      ok = r != 0;
    }
    flag[i] = ok;
  }
}

// ----------------------------------------------------------------------------- multi-exponentiation
// Pippenger bucket method for out_j = prod_{t in seg j} c[idx t]^(e_t): the exponent bits are
// cut into W windows of cb bits; bucket (j, w, v) collects the inputs whose window-w digit is v.

// segment of entry t (offsets non-decreasing, nseg >= 1)
__device__ __forceinline__ int64_t seg_of(const int64_t* __restrict__ off, int64_t nseg, int64_t t) {
  int64_t lo = 0, hi = nseg - 1;
  while (lo < hi) {
    const int64_t mid = (lo + hi + 1) >> 1;
    if (off[mid] <= t) lo = mid; else hi = mid - 1;
  }
  return lo;
}

__device__ __forceinline__ uint32_t exp_digit(const uint32_t* __restrict__ e, uint32_t e_words, uint32_t lo, uint32_t cb) {
  const uint32_t word = lo >> 5, off = lo & 31u;
  uint64_t v = (word < e_words) ? __ldg(e + word) : 0u;
  if (word + 1 < e_words) v |= (uint64_t)__ldg(e + word + 1) << 32;
  return (uint32_t)(v >> off) & ((1u << cb) - 1u);
}

// pass 0: count bucket sizes; pass 1: scatter input indices into buckets (cursor = bucket starts)
template <int PASS>
__global__ void k_bucket(const int64_t* __restrict__ off, int64_t nseg, int64_t nent, const int64_t* __restrict__ idx,
                         const uint32_t* __restrict__ e, uint32_t e_words, uint32_t W, uint32_t cb,
                         unsigned long long* __restrict__ cnt_or_cursor, int64_t* __restrict__ sorted) {
  for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < nent; t += (int64_t)gridDim.x * blockDim.x) {
    const int64_t j = seg_of(off, nseg, t);
    const uint32_t* et = e + t * e_words;
    for (uint32_t w = 0; w < W; w++) {
      const uint32_t v = exp_digit(et, e_words, w * cb, cb);
      if (!v) continue;
      const uint64_t b = ((uint64_t)j * W + w) << cb | v;
      if (PASS == 0) {
        atomicAdd(cnt_or_cursor + b, 1ull);
      } else {
        const unsigned long long pos = atomicAdd(cnt_or_cursor + b, 1ull);
        sorted[pos] = idx ? idx[t] : t;
      }
    }
  }
}

// exclusive scan of n counters (one block): out[i] = sum_{k<i} in[k], out[n] = total
static __global__ void k_scan_u64(const unsigned long long* __restrict__ in, int64_t n, int64_t* __restrict__ out) {
  __shared__ long long warp_sums[32];
  __shared__ long long carry;
  if (threadIdx.x == 0) carry = 0;
  __syncthreads();
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  for (int64_t base = 0; base < n; base += blockDim.x) {
    const int64_t i = base + threadIdx.x;
    const long long v = i < n ? (long long)in[i] : 0;
    long long x = v;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const long long y = __shfl_up_sync(FULL, x, o);
      if (lane >= o) x += y;
    }
    if (lane == 31) warp_sums[wid] = x;
    __syncthreads();
    if (wid == 0) {
      long long s = (lane < (int)(blockDim.x >> 5)) ? warp_sums[lane] : 0;
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const long long y = __shfl_up_sync(FULL, s, o);
        if (lane >= o) s += y;
      }
      warp_sums[lane] = s;
    }
    __syncthreads();
    const long long before = carry + (wid ? warp_sums[wid - 1] : 0) + x - v;
    if (i < n) out[i] = before;
    __syncthreads();
    if (threadIdx.x == blockDim.x - 1) carry = before + v;
    __syncthreads();
  }
  if (threadIdx.x == 0) out[n] = carry;
}

// bit-plane index: for plane p = (j, w, bit) list the buckets (j, w, v) with that bit of v set
static __global__ void k_bitplane_index(int64_t nplanes, uint32_t cb, int64_t* __restrict__ idx2) {
  const int64_t half = (int64_t)1 << (cb - 1);
  const int64_t total = nplanes * half;
  for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < total; t += (int64_t)gridDim.x * blockDim.x) {
    const int64_t p = t / half, r = t - p * half;
    const uint32_t bit = (uint32_t)(p % cb);
    const int64_t jw = p / cb;
    // r-th value v in [1, 2^cb) with bit `bit` set: insert a 1 at position `bit` into r
    const uint64_t low = (uint64_t)r & ((1ull << bit) - 1), high = ((uint64_t)r >> bit) << (bit + 1);
    const uint64_t v = high | (1ull << bit) | low;
    idx2[t] = (jw << cb) | (int64_t)v;
  }
}

static __global__ void k_arange_offsets(int64_t n, int64_t step, int64_t* __restrict__ out) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i <= n; i += (int64_t)gridDim.x * blockDim.x)
    out[i] = i * step;
}

struct HornerArgs {
  ModRef N2;
  const uint32_t* R1;
  const uint32_t* R2;
  const uint32_t* P;   // [nseg][K][S] bit-plane products (plane k = w * cb + bit)
  uint32_t K;
  uint32_t* out;       // [nseg][S]
  uint64_t nseg;
};

// out_j = prod_k P_{j,k}^(2^k) by Horner from the top bit (Montgomery domain inside).
template <int X, int T>
__global__ void __launch_bounds__(32, FLB_MINB_MUL) k_horner(const HornerArgs A) {
  constexpr int S = X * T;
  const Grid<T> g;
  uint32_t n[X];
  load_mod<X, T>(n, A.N2);
  const uint32_t n0inv = A.N2.n0inv;
  for (uint64_t base = g.wg0; base < A.nseg; base += g.G) {
    const uint64_t j = base + (g.gid - g.wg0);
    const bool valid = j < A.nseg;
    uint32_t acc[X], b[X], r2[X];
    load_const<X, T>(acc, A.R1);
    load_const<X, T>(r2, A.R2);
#pragma unroll 1
    for (int k = (int)A.K - 1; k >= 0; k--) {
      mont_sqr<X, T>(acc, acc, n, n0inv);
      load_elem<X, T>(b, A.P + (j * A.K + (uint64_t)k) * S, S, valid);
      mont_mul<X, T>(b, b, r2, n, n0inv);
      mont_mul<X, T>(acc, acc, b, n, n0inv);
    }
    set_one<X, T>(b);
    mont_mul<X, T>(acc, acc, b, n, n0inv);
    if (valid) store_limbs<X>(A.out + j * S + g.k * X, acc);
  }
}

// rows[i] = c[idx[i]] (gather, one thread per word)
static __global__ void k_gather_rows(const uint32_t* __restrict__ c, const int64_t* __restrict__ idx, int64_t n, uint32_t S,
                              uint32_t* __restrict__ out) {
  const int64_t total = n * S;
  for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < total; t += (int64_t)gridDim.x * blockDim.x) {
    const int64_t i = t / S;
    out[t] = c[(idx ? idx[i] : i) * S + (t - i * S)];
  }
}

// ----------------------------------------------------------------------------- key-holder encrypt, v2
// r^n mod P^2 = ((r^Q mod P))^P mod P^2 for {P, Q} = {p, q}: x^P mod P^2 depends only on x mod P
// ((y + kP)^P = y^P mod P^2 by the binomial theorem), and r^n = (r^Q)^P.  Stage 1 (this kernel,
// half-size frame): y_P = r^Q mod P.  Stage 2 (k_encrypt_crt2, P^2 frame): c_P = (1 + mn) y_P^P
// mod P^2, then the CRT combine of k_encrypt_crt.  Exact for every r (r = 0 mod P gives 0 both ways).
struct CrtPreArgs {
  ModRef P[2];             // p, q in the half frame
  const uint32_t* R2[2];   // R^2 mod P (half frame)
  const uint32_t* R3[2];   // R^3 mod P
  const uint32_t* sched[2];  // exponent Q (the other prime) for P
  int sched_len[2], table[2];
  uint32_t nbits;          // bits(n)
  uint32_t pt_words;       // sp (the frame of r)
  const uint32_t* r;       // [count][pt_words] or null (Philox)
  uint64_t seed, ctr0;
  uint32_t* y;             // [2][count][H]
  uint64_t count;
  uint32_t* scratch;
};

template <int X, int T>
__global__ void __launch_bounds__(32, FLB_MINB_DEC) k_crt_pre(const CrtPreArgs A) {
  constexpr int H = X * T;
  const Grid<T> g;
  uint32_t* tab = A.scratch + (size_t)g.gid * H;
  const size_t stride = (size_t)g.G * H;
  for (uint64_t base = g.wg0; base < A.count; base += g.G) {
    const uint64_t e = base + (g.gid - g.wg0);
    const bool valid = e < A.count;
#pragma unroll 1
    for (int P = 0; P < 2; P++) {
      uint32_t n[X], lo[X], hi[X], b[X], x[X];
      load_mod<X, T>(n, A.P[P]);
      const uint32_t n0inv = A.P[P].n0inv;
      if (A.r) {
        load_elem<X, T>(lo, A.r + e * A.pt_words, min(A.pt_words, (uint32_t)H), valid);
        if (A.pt_words > (uint32_t)H) load_elem<X, T>(hi, A.r + e * A.pt_words + H, A.pt_words - H, valid);
        else zero_limbs<X>(hi);
      } else {
        // the same words philox_r draws for the whole r: low H words, then the rest; r = 0 -> 1
        philox_r<X, T>(lo, A.seed, A.ctr0 + e, A.pt_words, A.nbits, 0, false);
        philox_r<X, T>(hi, A.seed, A.ctr0 + e, A.pt_words, A.nbits, H, false);
        const bool nz = !(all_zero<X>(lo) && all_zero<X>(hi));
        const uint32_t bal = __ballot_sync(FULL, nz);
        const int gb = (T == 32) ? 0 : (int)(lane_id() & ~(uint32_t)(T - 1));
        const uint32_t gm = (T == 32) ? 0xffffffffu : (((1u << T) - 1u) << gb);
        if ((bal & gm) == 0 && g.k == 0) lo[0] = 1;
      }
      load_const<X, T>(b, A.R2[P]);
      mont_mul<X, T>(lo, lo, b, n, n0inv);                   // r_lo R mod P
      load_const<X, T>(b, A.R3[P]);
      mont_mul<X, T>(hi, hi, b, n, n0inv);                   // r_hi R^2 mod P
      const uint32_t cy = grp_add<X, T>(x, lo, hi);
      grp_cond_sub<X, T>(x, n, cy);                          // r R mod P
      modexp_sched<X, T>(lo, x, A.sched[P], A.sched_len[P], A.table[P], tab, stride, n, n0inv);
      set_one<X, T>(b);
      mont_mul<X, T>(lo, lo, b, n, n0inv);                   // y_P = r^Q mod P
      if (valid) store_limbs<X>(A.y + ((uint64_t)P * A.count + e) * H + g.k * X, lo);
    }
  }
}

struct EncCrt2Args {
  ModRef P2[2];
  const uint32_t* R2[2];   // R^2 mod P^2 (sp frame)
  const uint32_t* nR[2];
  const uint32_t* q2;
  const uint32_t* q2invR;
  const uint32_t* sched[2];  // exponent P for P^2
  int sched_len[2], table[2];
  const uint32_t* m;       // [count][sp]
  const uint32_t* y;       // [2][count][H]
  uint32_t H;
  uint32_t* c;             // [count][2 sp]
  uint64_t count;
  uint32_t* scratch;
};

template <int X, int T>
__global__ void __launch_bounds__(32, FLB_MINB_DEC) k_encrypt_crt2(const EncCrt2Args A) {
  constexpr int S = X * T;  // sp
  const Grid<T> g;
  uint32_t* tab = A.scratch + (size_t)g.gid * S;
  const size_t stride = (size_t)g.G * S;
  for (uint64_t base = g.wg0; base < A.count; base += g.G) {
    const uint64_t e = base + (g.gid - g.wg0);
    const bool valid = e < A.count;
    uint32_t cres[2][X];
#pragma unroll 1
    for (int P = 0; P < 2; P++) {
      uint32_t n[X], x[X], b[X], acc[X];
      load_mod<X, T>(n, A.P2[P]);
      const uint32_t n0inv = A.P2[P].n0inv;
      load_elem<X, T>(x, A.y + ((uint64_t)P * A.count + e) * A.H, A.H, valid);
      load_const<X, T>(b, A.R2[P]);
      mont_mul<X, T>(x, x, b, n, n0inv);                       // y R mod P^2
      modexp_sched<X, T>(acc, x, A.sched[P], A.sched_len[P], A.table[P], tab, stride, n, n0inv);  // y^P R
      load_elem<X, T>(x, A.m + e * S, S, valid);
      load_const<X, T>(b, A.nR[P]);
      mont_mul<X, T>(x, x, b, n, n0inv);                       // m n mod P^2
      set_one<X, T>(b);
      const uint32_t cy = grp_add<X, T>(x, x, b);
      grp_cond_sub<X, T>(x, n, cy);                            // 1 + m n mod P^2
      mont_mul<X, T>(acc, acc, x, n, n0inv);                   // c_P = (1 + mn) r^n mod P^2
#pragma unroll
      for (int j = 0; j < X; j++) {
        if (P == 0) cres[0][j] = acc[j];
        else cres[1][j] = acc[j];
      }
    }
    uint32_t n[X], d[X], t[X], hi[X];
    load_mod<X, T>(n, A.P2[0]);
    const uint32_t br = grp_sub<X, T>(d, cres[0], cres[1]);
#pragma unroll
    for (int j = 0; j < X; j++) t[j] = br ? n[j] : 0u;
    grp_add<X, T>(d, d, t);
    load_const<X, T>(t, A.q2invR);
    mont_mul<X, T>(d, d, t, n, A.P2[0].n0inv);
    load_const<X, T>(t, A.q2);
    mul_full<X, T>(d, hi, d, t);
    const uint32_t cy = grp_add<X, T>(d, d, cres[1]);
    grp_add_small<X, T>(hi, cy);
    if (valid) {
      store_limbs<X>(A.c + e * (2 * S) + g.k * X, d);
      store_limbs<X>(A.c + e * (2 * S) + S + g.k * X, hi);
    }
  }
}

// ----------------------------------------------------------------------------- hom-add
struct AddArgs {
  ModRef N2;
  const uint32_t* R2;
  const uint32_t* c1;
  const uint32_t* c2;
  uint32_t* out;
  uint64_t count;
};

// c1 c2 mod n^2 (Eq. 5) = mont(mont(c1, c2), R^2).
template <int X, int T>
__global__ void __launch_bounds__(32, FLB_MINB_MUL) k_add(const AddArgs A) {
  constexpr int S = X * T;
  const Grid<T> g;
  uint32_t n[X];
  load_mod<X, T>(n, A.N2);
  for (uint64_t base = g.wg0; base < A.count; base += g.G) {
    const uint64_t e = base + (g.gid - g.wg0);
    const bool valid = e < A.count;
    uint32_t a[X], b[X];
    load_elem<X, T>(a, A.c1 + e * S, S, valid);
    load_elem<X, T>(b, A.c2 + e * S, S, valid);
#pragma unroll 1
    for (int it = 0; it < 2; it++) {
      mont_mul<X, T>(a, a, b, n, A.N2.n0inv);
      load_const<X, T>(b, A.R2);
    }
    if (valid) store_limbs<X>(A.out + e * S + g.k * X, a);
  }
}

// ----------------------------------------------------------------------------- debug mont_mul
template <int X, int T>
__global__ void __launch_bounds__(32, FLB_MINB_MUL) k_mont(const AddArgs A) {
  constexpr int S = X * T;
  const Grid<T> g;
  uint32_t n[X];
  load_mod<X, T>(n, A.N2);
  for (uint64_t base = g.wg0; base < A.count; base += g.G) {
    const uint64_t e = base + (g.gid - g.wg0);
    const bool valid = e < A.count;
    uint32_t a[X], b[X];
    load_elem<X, T>(a, A.c1 + e * S, S, valid);
    load_elem<X, T>(b, A.c2 + e * S, S, valid);
    mont_mul<X, T>(a, a, b, n, A.N2.n0inv);
    if (valid) store_limbs<X>(A.out + e * S + g.k * X, a);
  }
}

// ----------------------------------------------------------------------------- scalar-mul
struct SmulArgs {
  ModRef N2;
  const uint32_t* R2;      // R^2 mod n^2
  const uint32_t* R1;      // R mod n^2 (Montgomery one)
  const uint32_t* c;       // [count][S]
  const uint32_t* e;       // [count][e_words]
  uint32_t e_words;
  int bw;                  // fixed window width
  uint32_t* out;
  uint64_t count;
  uint32_t* scratch;       // 2^bw * G * S
};

__device__ __forceinline__ uint32_t exp_window(const uint32_t* e, uint32_t e_words, int w, int bw) {
  const uint32_t lo = (uint32_t)(w * bw), word = lo >> 5, off = lo & 31u;
  uint32_t v = (word < e_words) ? __ldg(e + word) >> off : 0u;
  if (off + bw > 32 && word + 1 < e_words) v |= __ldg(e + word + 1) << (32 - off);
  return v & ((1u << bw) - 1u);
}

// c^e mod n^2 (mod_pow; reading c19), per-element exponent, fixed window with
// an always-multiply step (table[0] = Montgomery one) so control flow is uniform.
template <int X, int T>
__global__ void __launch_bounds__(32, FLB_MINB_ENC) k_scalar_mul(const SmulArgs A) {
  constexpr int S = X * T;
  const Grid<T> g;
  uint32_t n[X];
  load_mod<X, T>(n, A.N2);
  const uint32_t n0inv = A.N2.n0inv;
  uint32_t* tab = A.scratch + (size_t)g.gid * S;
  const size_t stride = (size_t)g.G * S;
  const int table = 1 << A.bw;
  for (uint64_t base = g.wg0; base < A.count; base += g.G) {
    const uint64_t el = base + (g.gid - g.wg0);
    const bool valid = el < A.count;
    uint32_t x[X], b[X], acc[X];
    load_elem<X, T>(x, A.c + el * S, S, valid);
    load_const<X, T>(b, A.R2);
    mont_mul<X, T>(x, x, b, n, n0inv);
    load_const<X, T>(acc, A.R1);
    store_limbs<X>(tab + g.k * X, acc);
    store_limbs<X>(tab + stride + g.k * X, x);
#pragma unroll
    for (int j = 0; j < X; j++) b[j] = x[j];
#pragma unroll 1
    for (int i = 2; i < table; i++) {
      mont_mul<X, T>(b, b, x, n, n0inv);
      store_limbs<X>(tab + (size_t)i * stride + g.k * X, b);
    }
    // highest window holding a set bit, maximised over the warp (uniform trip count)
    const uint32_t* ep = A.e + el * A.e_words;
    int top = -1;
    if (valid) {
      for (int w = (int)A.e_words - 1; w >= 0; w--) {
        const uint32_t v = __ldg(ep + w);
        if (v) { top = (int)((32 * w + 31 - __clz(v)) / A.bw); break; }
      }
    }
    top = __reduce_max_sync(FULL, top);
#pragma unroll 1
    for (int w = top; w >= 0; w--) {
      if (w != top) {
#pragma unroll 1
        for (int s = 0; s < A.bw; s++) mont_sqr<X, T>(acc, acc, n, n0inv);
      }
      const uint32_t d = valid ? exp_window(ep, A.e_words, w, A.bw) : 0u;
      load_limbs_plain<X>(b, tab + (size_t)d * stride + g.k * X);
      mont_mul<X, T>(acc, acc, b, n, n0inv);
    }
    set_one<X, T>(b);
    mont_mul<X, T>(acc, acc, b, n, n0inv);
    if (valid) store_limbs<X>(A.out + el * S + g.k * X, acc);
  }
}

// ----------------------------------------------------------------------------- segmented reduce
struct RedArgs {
  ModRef N2;
  const uint32_t* R1;          // R mod n^2
  const uint32_t* RL;          // R^L mod n^2 for L = 0..C, [C+1][S]
  const uint32_t* in;          // [*][S]
  const int64_t* idx;          // gather index into `in` or null
  const int64_t* cstart;       // per chunk: first input position
  const int64_t* cend;         // per chunk: one past the last
  const int64_t* nchunks;      // device scalar: number of chunks
  uint32_t* out;               // [nchunks][S]
  uint64_t max_chunks;         // host bound for the grid
};

// out[ch] = prod_{t in chunk} in[idx[t]] mod n^2.  acc starts at R (Montgomery one); after L
// raw-input Montgomery products it is prod * R^-(L-1); one product with R^L mod n^2 removes the
// factor.  Lanes whose chunk is shorter multiply by R mod n^2 (a no-op).
template <int X, int T>
__global__ void __launch_bounds__(32, FLB_MINB_MUL) k_reduce(const RedArgs A) {
  constexpr int S = X * T;
  const Grid<T> g;
  uint32_t n[X];
  load_mod<X, T>(n, A.N2);
  const uint64_t count = (uint64_t)*A.nchunks;
  for (uint64_t base = g.wg0; base < count; base += g.G) {
    const uint64_t ch = base + (g.gid - g.wg0);
    const bool valid = ch < count;
    int64_t st = 0, len = 0;
    if (valid) { st = A.cstart[ch]; len = A.cend[ch] - st; }
    const int maxlen = __reduce_max_sync(FULL, (int)len);
    uint32_t acc[X], b[X];
    load_const<X, T>(acc, A.R1);
#pragma unroll 1
    for (int t = 0; t <= maxlen; t++) {
      if (t < maxlen) {
        if (t < len) {
          const int64_t pos = A.idx ? A.idx[st + t] : st + t;
          load_limbs<X>(b, A.in + (size_t)pos * S + g.k * X);
        } else {
          load_const<X, T>(b, A.R1);
        }
      } else {
        load_const<X, T>(b, A.RL + (size_t)len * S);
      }
      mont_mul<X, T>(acc, acc, b, n, A.N2.n0inv);
    }
    if (valid) store_limbs<X>(A.out + ch * S + g.k * X, acc);
  }
}

// chunk planning: chunks_j = max(1, ceil(len_j / C)); chunk_off = exclusive scan (one block).
static __global__ void k_plan_scan(const int64_t* __restrict__ offsets, int64_t nseg, int C, int64_t* __restrict__ chunk_off) {
  __shared__ int64_t warp_sums[32];
  __shared__ int64_t carry;
  if (threadIdx.x == 0) carry = 0;
  __syncthreads();
  for (int64_t base = 0; base < nseg; base += blockDim.x) {
    const int64_t j = base + threadIdx.x;
    int64_t v = 0;
    if (j < nseg) {
      const int64_t len = offsets[j + 1] - offsets[j];
      v = len <= 0 ? 1 : (len + C - 1) / C;
    }
    // inclusive warp scan
    int64_t x = v;
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const int64_t y = __shfl_up_sync(FULL, x, o);
      if (lane >= o) x += y;
    }
    if (lane == 31) warp_sums[wid] = x;
    __syncthreads();
    if (wid == 0) {
      int64_t s = (lane < (int)(blockDim.x >> 5)) ? warp_sums[lane] : 0;
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const int64_t y = __shfl_up_sync(FULL, s, o);
        if (lane >= o) s += y;
      }
      warp_sums[lane] = s;  // inclusive over warps
    }
    __syncthreads();
    const int64_t before = carry + (wid ? warp_sums[wid - 1] : 0) + x - v;
    if (j < nseg) chunk_off[j] = before;
    __syncthreads();
    if (threadIdx.x == blockDim.x - 1) carry = before + v;
    __syncthreads();
  }
  if (threadIdx.x == 0) chunk_off[nseg] = carry;
}

static __global__ void k_plan_fill(const int64_t* __restrict__ offsets, const int64_t* __restrict__ chunk_off, int64_t nseg,
                            int C, int64_t* __restrict__ cstart, int64_t* __restrict__ cend) {
  const int64_t total = chunk_off[nseg];
  for (int64_t c = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; c < total; c += (int64_t)gridDim.x * blockDim.x) {
    // segment j: last j with chunk_off[j] <= c
    int64_t lo = 0, hi = nseg - 1;
    while (lo < hi) {
      const int64_t mid = (lo + hi + 1) >> 1;
      if (chunk_off[mid] <= c) lo = mid; else hi = mid - 1;
    }
    const int64_t j = lo, r = c - chunk_off[j];
    const int64_t s = offsets[j] + r * C;
    int64_t e = s + C;
    if (e > offsets[j + 1]) e = offsets[j + 1];
    if (e < s) e = s;
    cstart[c] = s;
    cend[c] = e;
  }
}

// ----------------------------------------------------------------------------- codec
struct CodecArgs {
  double alpha, sigma;
  uint32_t qbits, slot_words, slots, pt_words;
  uint64_t qmax;
};

// Eq. 6–7 in binary64, op for op as oracle/codec.py quantize (reading c11, c13).
__device__ __forceinline__ uint64_t quantize(float xf, const CodecArgs& C) {
  double x = (double)xf;
  if (isnan(x)) x = 0.0;
  x = fmin(fmax(x, -C.alpha), C.alpha);
  const double e = __dadd_rn(x, C.alpha);
  const double p = __dmul_rn(e, C.sigma);
  double q = rint(p);
  if (q < 0.0) q = 0.0;
  uint64_t qi = (uint64_t)q;
  return qi > C.qmax ? C.qmax : qi;
}

// pt[j] = sum_i q_{jS+i} 2^((S-1-i) w) (Eq. 9, reading c17); one thread per word.
static __global__ void k_pack(const float* __restrict__ x, uint64_t n_values, uint64_t n_pt, CodecArgs C,
                       uint32_t* __restrict__ pt) {
  const uint64_t total = n_pt * C.pt_words;
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < total; i += (uint64_t)gridDim.x * blockDim.x) {
    const uint64_t j = i / C.pt_words;
    const uint32_t t = (uint32_t)(i - j * C.pt_words);
    uint32_t w = 0;
    if (t < C.slots * C.slot_words) {
      const uint32_t slot = C.slots - 1 - t / C.slot_words, part = t % C.slot_words;
      const uint64_t v = j * C.slots + slot;
      if (v < n_values && part < 2) w = (uint32_t)(quantize(x[v], C) >> (32 * part));
    }
    pt[i] = w;
  }
}

__device__ __forceinline__ uint64_t slot_value(const uint32_t* __restrict__ pt, uint64_t v, const CodecArgs& C) {
  const uint64_t j = v / C.slots;
  const uint32_t i = (uint32_t)(v - j * C.slots);
  const uint32_t w0 = (C.slots - 1 - i) * C.slot_words;
  const uint32_t* p = pt + j * C.pt_words + w0;
  uint64_t s = p[0];
  if (C.slot_words > 1) s |= (uint64_t)p[1] << 32;
  return s;
}

// x = Sum / sigma - cnt alpha in binary64, then binary32 (reading c14).
static __global__ void k_unpack(const uint32_t* __restrict__ pt, uint64_t n_values, CodecArgs C,
                         const uint32_t* __restrict__ summands, uint32_t summands_scalar, float* __restrict__ out) {
  for (uint64_t v = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; v < n_values; v += (uint64_t)gridDim.x * blockDim.x) {
    const uint64_t s = slot_value(pt, v, C);
    const uint32_t cnt = summands ? summands[v / C.slots] : summands_scalar;
    const double t1 = __ddiv_rn(__ull2double_rn(s), C.sigma);
    const double t2 = __dmul_rn((double)cnt, C.alpha);
    out[v] = __double2float_rn(__dsub_rn(t1, t2));
  }
}

static __global__ void k_unpack_sums(const uint32_t* __restrict__ pt, uint64_t n_values, CodecArgs C,
                              unsigned long long* __restrict__ out) {
  for (uint64_t v = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; v < n_values; v += (uint64_t)gridDim.x * blockDim.x)
    out[v] = slot_value(pt, v, C);
}

}  // namespace flb

namespace flb {
// ----------------------------------------------------------------------------- CRT combine
// c = c_q + q^2 ((c_p - c_q) (q^2)^-1 mod p^2) from c_p = c mod p^2, c_q = c mod q^2 (the combine
// step of k_encrypt_crt2, for stage-2 results computed elsewhere, e.g. by the tensor-core kernel).
struct CombineArgs {
  ModRef P2;               // p^2 in the sp frame
  const uint32_t* q2;      // q^2 (sp limbs, plain)
  const uint32_t* q2invR;  // (q^2)^-1 R mod p^2
  const uint32_t* cp;      // [count][sp]
  const uint32_t* cq;      // [count][sp]
  uint32_t* c;             // [count][2 sp]
  uint64_t count;
};

template <int X, int T>
__global__ void __launch_bounds__(32, FLB_MINB_MUL) k_crt_combine(const CombineArgs A) {
  constexpr int S = X * T;
  const Grid<T> g;
  for (uint64_t base = g.wg0; base < A.count; base += g.G) {
    const uint64_t e = base + (g.gid - g.wg0);
    const bool valid = e < A.count;
    uint32_t n[X], d[X], t[X], hi[X], cp[X], cq[X];
    load_elem<X, T>(cp, A.cp + e * S, S, valid);
    load_elem<X, T>(cq, A.cq + e * S, S, valid);
    load_mod<X, T>(n, A.P2);
    const uint32_t br = grp_sub<X, T>(d, cp, cq);
#pragma unroll
    for (int j = 0; j < X; j++) t[j] = br ? n[j] : 0u;
    grp_add<X, T>(d, d, t);
    load_const<X, T>(t, A.q2invR);
    mont_mul<X, T>(d, d, t, n, A.P2.n0inv);
    load_const<X, T>(t, A.q2);
    mul_full<X, T>(d, hi, d, t);
    const uint32_t cy = grp_add<X, T>(d, d, cq);
    grp_add_small<X, T>(hi, cy);
    if (valid) {
      store_limbs<X>(A.c + e * (2 * S) + g.k * X, d);
      store_limbs<X>(A.c + e * (2 * S) + S + g.k * X, hi);
    }
  }
}
// The CRT tail of k_decrypt after the two exponentiations (done on the tensor cores, flb_tc.cuh
// k_tc_exp): from x_P = c^(P-1) mod P^2, m_P = L_P(x_P) h_P mod P and
// m = m_q + q ((m_p - m_q) q^-1 mod p) (Eq. 4 by CRT, reading c10).
template <int X, int T>
__global__ void __launch_bounds__(32, FLB_MINB_MUL) k_dec_finish(const DecArgs A) {
  constexpr int S = X * T;  // sp
  const Grid<T> g;
  for (uint64_t base = g.wg0; base < A.count; base += g.G) {
    const uint64_t e = base + (g.gid - g.wg0);
    const bool valid = e < A.count;
    uint32_t mres[2][X];
#pragma unroll 1
    for (int P = 0; P < 2; P++) {
      const PrimeArgs& pa = A.pr[P];
      uint32_t n[X], lo[X], hi[X], b[X];
      load_elem<X, T>(lo, A.xp + ((uint64_t)P * A.count + e) * S, S, valid);
      grp_sub_one<X, T>(lo);                              // x - 1 = L * P
      load_const<X, T>(b, pa.Pinv);
      mul_lo<X, T>(hi, lo, b);                            // L = (x - 1) / P (exact division)
      load_mod<X, T>(n, pa.P);
      load_const<X, T>(b, pa.hR);
      mont_mul<X, T>(lo, hi, b, n, pa.P.n0inv);           // m_P = L h_P mod P
#pragma unroll
      for (int j = 0; j < X; j++) {
        if (P == 0) mres[0][j] = lo[j];
        else mres[1][j] = lo[j];
      }
    }
    uint32_t n[X], d[X], t[X];
    load_mod<X, T>(n, A.pr[0].P);
    const uint32_t br = grp_sub<X, T>(d, mres[0], mres[1]);   // m_p - m_q (m_q < q < p)
#pragma unroll
    for (int j = 0; j < X; j++) t[j] = br ? n[j] : 0u;
    grp_add<X, T>(d, d, t);                                    // mod p
    load_const<X, T>(t, A.qinvR_p);
    mont_mul<X, T>(d, d, t, n, A.pr[0].P.n0inv);               // u = (m_p - m_q) q^-1 mod p
    load_mod<X, T>(n, A.n);
    load_const<X, T>(t, A.qR_n);
    mont_mul<X, T>(d, d, t, n, A.n.n0inv);                     // q u (< n, exact)
    grp_add<X, T>(d, d, mres[1]);                              // m = m_q + q u
    if (valid) store_limbs<X>(A.m + e * S + g.k * X, d);
  }
}

// r for elements [0, count) as k_encrypt draws it (philox_r, reading c4) into [count][pt_words],
// X T = pt_words: the input of the tensor-core first stage of the key-holder encryption.
template <int X, int T>
__global__ void __launch_bounds__(32, FLB_MINB_MUL) k_philox_fill(uint32_t* __restrict__ r, uint64_t count,
                                                                  uint32_t nbits, uint64_t seed, uint64_t ctr0) {
  constexpr int S = X * T;
  const Grid<T> g;
  for (uint64_t base = g.wg0; base < count; base += g.G) {
    const uint64_t e = base + (g.gid - g.wg0);
    uint32_t v[X];
    philox_r<X, T>(v, seed, ctr0 + e, S, nbits);
    if (e < count) store_limbs<X>(r + e * S + g.k * X, v);
  }
}
}  // namespace flb

