// flb_bn.cuh — thread-group multi-precision arithmetic for sm_100a (layer L0).
//
// A big integer of S = X*T little-endian 32-bit limbs (§IV-A1: radix 2^w,
// w = 32, "each thread processes s/d limbs") is spread over a group of T consecutive lanes of
// one warp; lane k of the group holds limbs [k*X, k*X + X) in registers.  Groups tile the warp
// (T in {2,4,8,16,32}), so every collective below is a full-warp __shfl/__ballot with a width-T
// segment and no lane is ever inactive.
//
// Montgomery multiplication is the CIOS form of PAPER Algorithm 2 (L146–L205 §IV-A3), re-laid
// out for the B200 integer pipe:
//   * every 32x32->64 limb product is ONE `IMAD.WIDE.U32.X` (mad.lo.cc + madc.hi.cc fused by
//     ptxas), the measured half-rate FMA-heavy op (tools/imad_peak.cu: ~28-32 per clk per SM);
//   * products of even limbs accumulate into E (words 0..X), odd limbs into O (words 1..X+1),
//     so every carry chain runs over aligned register pairs and needs no separate add;
//   * the CIOS word shift (Alg. 2 lines 16–17) is register renaming (E' = O, O' = E >> 2 words)
//     plus one shuffle that moves each lane's lowest word to the lane below; carries that
//     cross lanes stay pending in two top words and are resolved once per multiplication with a
//     ballot-based carry-lookahead ("propagate the overflow ... via inter-thread
//     communication");
//   * outputs are canonical in [0, N) with a full compare-subtract (reading c8: Alg. 2's
//     "if t_{T-1} > 0" test alone leaves results in [N, R)).
// Reading c6/c7: n0inv = -N^-1 mod 2^32 and R = 2^(32*S).
#pragma once
#include <cstdint>

namespace flb {

constexpr unsigned FULL = 0xffffffffu;

__device__ __forceinline__ uint32_t lane_id() { return threadIdx.x & 31u; }

// ----------------------------------------------------------------------------- carry lookahead
// Carry into every lane of the group given per-lane generate g / propagate p (mutually
// exclusive) and a carry-in to lane 0.  c_i = g_{i-1} | (p_{i-1} & c_{i-1}), computed as
// ((p|g) + g + cin) ^ p over the group's ballot bits.  Returns the lane's carry-in in bit 0 and
// the group's carry-out (carry out of lane T-1) in bit 1.
template <int T>
__device__ __forceinline__ uint32_t group_carry(bool g, bool p, uint32_t cin) {
  const uint32_t G = __ballot_sync(FULL, g), P = __ballot_sync(FULL, p);
  const int base = (T == 32) ? 0 : (int)(lane_id() & ~(uint32_t)(T - 1));
  const uint64_t mask = (T == 32) ? 0xffffffffull : ((1ull << T) - 1);
  const uint64_t gg = ((uint64_t)G >> base) & mask, pp = ((uint64_t)P >> base) & mask;
  const uint64_t c = ((pp | gg) + gg + cin) ^ pp;
  const int k = (int)(lane_id() & (T - 1));
  return (uint32_t)((c >> k) & 1u) | ((uint32_t)((c >> T) & 1u) << 1);
}

// ----------------------------------------------------------------------------- limb helpers
template <int X>
__device__ __forceinline__ uint32_t add_word_propagate(uint32_t (&r)[X], uint32_t v) {
  // r += v (v at word 0), returns carry out
  uint32_t c;
  asm volatile("add.cc.u32 %0, %0, %1;" : "+r"(r[0]) : "r"(v));
#pragma unroll
  for (int j = 1; j < X; j++) asm volatile("addc.cc.u32 %0, %0, 0;" : "+r"(r[j]));
  asm volatile("addc.u32 %0, 0, 0;" : "=r"(c));
  return c;
}

template <int X>
__device__ __forceinline__ bool all_ones(const uint32_t (&r)[X]) {
  uint32_t a = r[0];
#pragma unroll
  for (int j = 1; j < X; j++) a &= r[j];
  return a == 0xffffffffu;
}

template <int X>
__device__ __forceinline__ bool all_zero(const uint32_t (&r)[X]) {
  uint32_t a = r[0];
#pragma unroll
  for (int j = 1; j < X; j++) a |= r[j];
  return a == 0u;
}

// r = a + b over the whole group (+ cin); returns the group carry-out (same in every lane).
template <int X, int T>
__device__ __forceinline__ uint32_t grp_add(uint32_t (&r)[X], const uint32_t (&a)[X],
                                            const uint32_t (&b)[X], uint32_t cin = 0) {
  uint32_t g;
  asm volatile("add.cc.u32 %0, %1, %2;" : "=r"(r[0]) : "r"(a[0]), "r"(b[0]));
#pragma unroll
  for (int j = 1; j < X; j++) asm volatile("addc.cc.u32 %0, %1, %2;" : "=r"(r[j]) : "r"(a[j]), "r"(b[j]));
  asm volatile("addc.u32 %0, 0, 0;" : "=r"(g));
  const uint32_t c = group_carry<T>(g != 0, all_ones<X>(r), cin);
  add_word_propagate<X>(r, c & 1u);
  return c >> 1;
}

// r = a - b over the whole group; returns the group borrow-out (1 if a < b).
template <int X, int T>
__device__ __forceinline__ uint32_t grp_sub(uint32_t (&r)[X], const uint32_t (&a)[X],
                                            const uint32_t (&b)[X]) {
  uint32_t g;
  asm volatile("sub.cc.u32 %0, %1, %2;" : "=r"(r[0]) : "r"(a[0]), "r"(b[0]));
#pragma unroll
  for (int j = 1; j < X; j++) asm volatile("subc.cc.u32 %0, %1, %2;" : "=r"(r[j]) : "r"(a[j]), "r"(b[j]));
  asm volatile("subc.u32 %0, 0, 0;" : "=r"(g));  // 0xffffffff on borrow
  // a borrow-in to a lane whose difference is all-zero propagates
  const uint32_t c = group_carry<T>(g != 0, all_zero<X>(r), 0);
  // subtract the borrow-in
  const uint32_t bi = c & 1u;
  asm volatile("sub.cc.u32 %0, %0, %1;" : "+r"(r[0]) : "r"(bi));
#pragma unroll
  for (int j = 1; j < X; j++) asm volatile("subc.cc.u32 %0, %0, 0;" : "+r"(r[j]));
  return c >> 1;
}

// r = a + small (small < 2^32 at word 0 of the group)
template <int X, int T>
__device__ __forceinline__ void grp_add_small(uint32_t (&r)[X], uint32_t small) {
  const int k = (int)(lane_id() & (T - 1));
  const uint32_t g = add_word_propagate<X>(r, k == 0 ? small : 0u);
  const uint32_t c = group_carry<T>(g != 0, all_ones<X>(r), 0);
  add_word_propagate<X>(r, c & 1u);
}

// r = a - 1 for a >= 1
template <int X, int T>
__device__ __forceinline__ void grp_sub_one(uint32_t (&r)[X]) {
  const int k = (int)(lane_id() & (T - 1));
  uint32_t g;
  asm volatile("sub.cc.u32 %0, %0, %1;" : "+r"(r[0]) : "r"(k == 0 ? 1u : 0u));
#pragma unroll
  for (int j = 1; j < X; j++) asm volatile("subc.cc.u32 %0, %0, 0;" : "+r"(r[j]));
  asm volatile("subc.u32 %0, 0, 0;" : "=r"(g));
  const uint32_t c = group_carry<T>(g != 0, all_zero<X>(r), 0);
  const uint32_t bi = c & 1u;
  asm volatile("sub.cc.u32 %0, %0, %1;" : "+r"(r[0]) : "r"(bi));
#pragma unroll
  for (int j = 1; j < X; j++) asm volatile("subc.cc.u32 %0, %0, 0;" : "+r"(r[j]));
}

// Canonicalise: given t (group value, plus `over` = 1 if the true value is t + R), return
// t mod N assuming the true value is < 2N.
template <int X, int T>
__device__ __forceinline__ void grp_cond_sub(uint32_t (&t)[X], const uint32_t (&n)[X], uint32_t over) {
  uint32_t d[X];
  const uint32_t borrow = grp_sub<X, T>(d, t, n);
  const bool take = (over != 0) || (borrow == 0);
#pragma unroll
  for (int j = 0; j < X; j++) t[j] = take ? d[j] : t[j];
}

// ----------------------------------------------------------------------------- CIOS core
// acc += a_even*bi into E (pairs (E0,E1),(E2,E3),...) / a_odd*bi into O (pairs (O0,O1),...).
template <int X>
__device__ __forceinline__ void chain_even(uint32_t (&E)[X + 1], const uint32_t (&a)[X], uint32_t bi) {
  asm volatile("mad.lo.cc.u32 %0, %2, %3, %0;\n\tmadc.hi.cc.u32 %1, %2, %3, %1;"
               : "+r"(E[0]), "+r"(E[1]) : "r"(a[0]), "r"(bi));
#pragma unroll
  for (int j = 2; j < X; j += 2)
    asm volatile("madc.lo.cc.u32 %0, %2, %3, %0;\n\tmadc.hi.cc.u32 %1, %2, %3, %1;"
                 : "+r"(E[j]), "+r"(E[j + 1]) : "r"(a[j]), "r"(bi));
  asm volatile("addc.u32 %0, %0, 0;" : "+r"(E[X]));
}

// O chain; if CARRY_IN the first product consumes the carry flag set by the caller.
template <int X, bool CARRY_IN>
__device__ __forceinline__ void chain_odd(uint32_t (&O)[X + 1], const uint32_t (&a)[X], uint32_t bi) {
  if (CARRY_IN)
    asm volatile("madc.lo.cc.u32 %0, %2, %3, %0;\n\tmadc.hi.cc.u32 %1, %2, %3, %1;"
                 : "+r"(O[0]), "+r"(O[1]) : "r"(a[1]), "r"(bi));
  else
    asm volatile("mad.lo.cc.u32 %0, %2, %3, %0;\n\tmadc.hi.cc.u32 %1, %2, %3, %1;"
                 : "+r"(O[0]), "+r"(O[1]) : "r"(a[1]), "r"(bi));
#pragma unroll
  for (int j = 3; j < X; j += 2)
    asm volatile("madc.lo.cc.u32 %0, %2, %3, %0;\n\tmadc.hi.cc.u32 %1, %2, %3, %1;"
                 : "+r"(O[j - 1]), "+r"(O[j]) : "r"(a[j]), "r"(bi));
  asm volatile("addc.u32 %0, %0, 0;" : "+r"(O[X]));
}

// One CIOS step (PAPER Alg. 2 lines 3–17 for one word b_i of b):
//   acc += a*bi; [REDUCE] m = acc_word0 * n0inv; acc += m*N; acc >>= 32 (one word).
// State: E (words 0..X), O (words 1..X+1), pend (a word that belongs at word 0, merged at the
// start of the next step).  Returns the word shifted out of lane 0 (the product's word i when
// !REDUCE; zero when REDUCE).
template <int X, int T, bool REDUCE>
__device__ __forceinline__ uint32_t cios_step(uint32_t (&E)[X + 1], uint32_t (&O)[X + 1], uint32_t& pend,
                                              const uint32_t (&a)[X], uint32_t bi,
                                              const uint32_t (&n)[X], uint32_t n0inv) {
  const int k = (int)(lane_id() & (T - 1));
  // merge the pending word into word 0; its carry enters the O chain at word 1
  asm volatile("add.cc.u32 %0, %0, %1;" : "+r"(E[0]) : "r"(pend));
  chain_odd<X, true>(O, a, bi);
  chain_even<X>(E, a, bi);
  uint32_t out = 0;
  if (REDUCE) {
    const uint32_t m = __shfl_sync(FULL, E[0], 0, T) * n0inv;
    chain_even<X>(E, n, m);
    chain_odd<X, false>(O, n, m);
  } else {
    out = __shfl_sync(FULL, E[0], 0, T);
  }
  // shift right by one word
  uint32_t up = __shfl_down_sync(FULL, E[0], 1, T);
  if (k == T - 1) up = 0;
  pend = E[1];
  uint32_t nE[X + 1], nO[X + 1];
#pragma unroll
  for (int t = 0; t <= X; t++) nE[t] = O[t];
#pragma unroll
  for (int t = 0; t + 2 <= X; t++) nO[t] = E[t + 2];
  asm volatile("add.cc.u32 %0, %0, %1;" : "+r"(nO[X - 2]) : "r"(up));
  asm volatile("addc.u32 %0, 0, 0;" : "=r"(nO[X - 1]));
  nO[X] = 0;
#pragma unroll
  for (int t = 0; t <= X; t++) { E[t] = nE[t]; O[t] = nO[t]; }
  return out;
}

// Collapse (E, O, pend) into X words per lane, pushing the two overflow words to the next lane
// and resolving cross-lane carries.  Returns the group's overflow (bits above R) as 0/1 — for
// Montgomery outputs (< 2N < 2R) at most one bit.
template <int X, int T>
__device__ __forceinline__ uint32_t collapse(uint32_t (&r)[X], const uint32_t (&E)[X + 1],
                                             const uint32_t (&O)[X + 1], uint32_t pend) {
  const int k = (int)(lane_id() & (T - 1));
  uint32_t wX, wX1;
  asm volatile("add.cc.u32 %0, %1, %2;" : "=r"(r[0]) : "r"(E[0]), "r"(pend));
#pragma unroll
  for (int t = 1; t < X; t++) asm volatile("addc.cc.u32 %0, %1, %2;" : "=r"(r[t]) : "r"(E[t]), "r"(O[t - 1]));
  asm volatile("addc.cc.u32 %0, %1, %2;" : "=r"(wX) : "r"(E[X]), "r"(O[X - 1]));
  asm volatile("addc.u32 %0, %1, 0;" : "=r"(wX1) : "r"(O[X]));
  // lane k's words X, X+1 are lane k+1's words 0, 1
  uint32_t lo = __shfl_up_sync(FULL, wX, 1, T), hi = __shfl_up_sync(FULL, wX1, 1, T);
  if (k == 0) { lo = 0; hi = 0; }
  uint32_t g;
  asm volatile("add.cc.u32 %0, %0, %1;" : "+r"(r[0]) : "r"(lo));
  asm volatile("addc.cc.u32 %0, %0, %1;" : "+r"(r[1]) : "r"(hi));
#pragma unroll
  for (int t = 2; t < X; t++) asm volatile("addc.cc.u32 %0, %0, 0;" : "+r"(r[t]));
  asm volatile("addc.u32 %0, 0, 0;" : "=r"(g));
  const uint32_t c = group_carry<T>(g != 0, all_ones<X>(r), 0);
  add_word_propagate<X>(r, c & 1u);
  // overflow of the whole group: top lane's own words X, X+1 and the group carry-out
  const uint32_t topw = __shfl_sync(FULL, wX | wX1, T - 1, T);
  return ((c >> 1) | (topw != 0)) ? 1u : 0u;
}

// ----------------------------------------------------------------------------- operand staging
// The broadcast operand b of a multiplication is staged in shared memory: each CIOS step reads
// its word b_i with one LDS that every lane of the group hits at the same address (a broadcast),
// replacing a register-file copy of b plus a shuffle.  Lane k's chunk sits at k*LD with LD = X+4
// so the 16-byte stores of the T lanes hit distinct bank quads.  Blocks have <= kMaxWarps warps.
constexpr int kMaxWarps = 1;  // flb_api.cu launches one-warp blocks

template <int X>
__device__ __forceinline__ uint32_t* stage_base() {
  constexpr int LD = X + 4;
  __shared__ __align__(16) uint32_t buf[kMaxWarps * 32 * LD];
  return buf + (threadIdx.x >> 5) * (32 * LD);
}

// this group's staging buffer
template <int X, int T>
__device__ __forceinline__ uint32_t* stage_group() {
  constexpr int LD = X + 4;
  return stage_base<X>() + (int)(lane_id() & ~(uint32_t)(T - 1)) * LD;
}

template <int X, int T>
__device__ __forceinline__ void stage(const uint32_t (&b)[X]) {
  constexpr int LD = X + 4;
  const int k = (int)(lane_id() & (T - 1));
  uint4* q = reinterpret_cast<uint4*>(stage_group<X, T>() + k * LD);
  __syncwarp();
#pragma unroll
  for (int v = 0; v < X / 4; v++) q[v] = make_uint4(b[4 * v], b[4 * v + 1], b[4 * v + 2], b[4 * v + 3]);
  __syncwarp();
}

// r = a * b * R^-1 mod N, canonical, with b staged by stage<X,T>().  a < N (or any a < R when
// b < N).  r may alias a.
template <int X, int T>
__device__ __forceinline__ void mont_mul_staged(uint32_t (&r)[X], const uint32_t (&a)[X],
                                                const uint32_t (&n)[X], uint32_t n0inv) {
  constexpr int LD = X + 4;
  const uint32_t* bs = stage_group<X, T>();
  uint32_t E[X + 1], O[X + 1], pend = 0;
#pragma unroll
  for (int t = 0; t <= X; t++) { E[t] = 0; O[t] = 0; }
#pragma unroll 1
  for (int kk = 0; kk < T; kk++) {
    const uint32_t* row = bs + kk * LD;
#pragma unroll
    for (int jj = 0; jj < X; jj++) cios_step<X, T, true>(E, O, pend, a, row[jj], n, n0inv);
  }
  const uint32_t over = collapse<X, T>(r, E, O, pend);
  grp_cond_sub<X, T>(r, n, over);
}

template <int X, int T>
__device__ __forceinline__ void mont_mul(uint32_t (&r)[X], const uint32_t (&a)[X], const uint32_t (&b)[X],
                                         const uint32_t (&n)[X], uint32_t n0inv) {
  stage<X, T>(b);
  mont_mul_staged<X, T>(r, a, n, n0inv);
}


template <int X, int T>
__device__ __forceinline__ void mont_sqr(uint32_t (&r)[X], const uint32_t (&a)[X], const uint32_t (&n)[X],
                                         uint32_t n0inv) {
  stage<X, T>(a);
  mont_mul_staged<X, T>(r, a, n, n0inv);
}

// r = a * b mod 2^(32*S) (the low half of the plain product).
template <int X, int T>
__device__ __forceinline__ void mul_lo(uint32_t (&r)[X], const uint32_t (&a)[X], const uint32_t (&b)[X]) {
  constexpr int LD = X + 4;
  const int k = (int)(lane_id() & (T - 1));
  stage<X, T>(b);
  const uint32_t* bs = stage_group<X, T>();
  uint32_t E[X + 1], O[X + 1], pend = 0, res[X];
  const uint32_t dummy_n[X] = {};
#pragma unroll
  for (int t = 0; t <= X; t++) { E[t] = 0; O[t] = 0; }
#pragma unroll
  for (int t = 0; t < X; t++) res[t] = 0;
#pragma unroll 1
  for (int kk = 0; kk < T; kk++) {
    const uint32_t* row = bs + kk * LD;
#pragma unroll
    for (int jj = 0; jj < X; jj++) {
      const uint32_t w = cios_step<X, T, false>(E, O, pend, a, row[jj], dummy_n, 0u);
      if (k == kk) res[jj] = w;
    }
  }
#pragma unroll
  for (int t = 0; t < X; t++) r[t] = res[t];
}

// (lo, hi) = a * b, the full 2S-limb plain product (hi < R since a, b < R).
template <int X, int T>
__device__ __forceinline__ void mul_full(uint32_t (&lo)[X], uint32_t (&hi)[X], const uint32_t (&a)[X],
                                         const uint32_t (&b)[X]) {
  constexpr int LD = X + 4;
  const int k = (int)(lane_id() & (T - 1));
  stage<X, T>(b);
  const uint32_t* bs = stage_group<X, T>();
  uint32_t E[X + 1], O[X + 1], pend = 0, res[X];
  const uint32_t dummy_n[X] = {};
#pragma unroll
  for (int t = 0; t <= X; t++) { E[t] = 0; O[t] = 0; }
#pragma unroll
  for (int t = 0; t < X; t++) res[t] = 0;
#pragma unroll 1
  for (int kk = 0; kk < T; kk++) {
    const uint32_t* row = bs + kk * LD;
#pragma unroll
    for (int jj = 0; jj < X; jj++) {
      const uint32_t w = cios_step<X, T, false>(E, O, pend, a, row[jj], dummy_n, 0u);
      if (k == kk) res[jj] = w;
    }
  }
#pragma unroll
  for (int t = 0; t < X; t++) lo[t] = res[t];
  collapse<X, T>(hi, E, O, pend);
}

// ----------------------------------------------------------------------------- lane-local rows
// lane-local product row: acc += a * bi (no neighbour lanes), shift one word, return the word out
template <int X>
__device__ __forceinline__ uint32_t local_row(uint32_t (&E)[X + 1], uint32_t (&O)[X + 1], uint32_t& pend,
                                              const uint32_t (&a)[X], uint32_t bi) {
  asm volatile("add.cc.u32 %0, %0, %1;" : "+r"(E[0]) : "r"(pend));
  chain_odd<X, true>(O, a, bi);
  chain_even<X>(E, a, bi);
  const uint32_t out = E[0];
  pend = E[1];
  uint32_t nE[X + 1], nO[X + 1];
#pragma unroll
  for (int t = 0; t <= X; t++) nE[t] = O[t];
#pragma unroll
  for (int t = 0; t + 2 <= X; t++) nO[t] = E[t + 2];
  nO[X - 1] = 0;
  nO[X] = 0;
#pragma unroll
  for (int t = 0; t <= X; t++) { E[t] = nE[t]; O[t] = nO[t]; }
  return out;
}

// ----------------------------------------------------------------------------- loads / stores
template <int X>
__device__ __forceinline__ void load_limbs(uint32_t (&r)[X], const uint32_t* __restrict__ p) {
  static_assert(X % 4 == 0, "X must be a multiple of 4 for 16-byte loads");
  const uint4* q = reinterpret_cast<const uint4*>(p);
#pragma unroll
  for (int v = 0; v < X / 4; v++) {
    const uint4 u = __ldg(q + v);
    r[4 * v] = u.x; r[4 * v + 1] = u.y; r[4 * v + 2] = u.z; r[4 * v + 3] = u.w;
  }
}

template <int X>
__device__ __forceinline__ void load_limbs_plain(uint32_t (&r)[X], const uint32_t* p) {
  const uint4* q = reinterpret_cast<const uint4*>(p);
#pragma unroll
  for (int v = 0; v < X / 4; v++) {
    const uint4 u = q[v];
    r[4 * v] = u.x; r[4 * v + 1] = u.y; r[4 * v + 2] = u.z; r[4 * v + 3] = u.w;
  }
}

template <int X>
__device__ __forceinline__ void store_limbs(uint32_t* p, const uint32_t (&r)[X]) {
  uint4* q = reinterpret_cast<uint4*>(p);
#pragma unroll
  for (int v = 0; v < X / 4; v++) q[v] = make_uint4(r[4 * v], r[4 * v + 1], r[4 * v + 2], r[4 * v + 3]);
}

template <int X>
__device__ __forceinline__ void zero_limbs(uint32_t (&r)[X]) {
#pragma unroll
  for (int j = 0; j < X; j++) r[j] = 0;
}

}  // namespace flb
