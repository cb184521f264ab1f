// flb_mp.cu — Table I's fundamental multi-precision array operations (Table I:
// add/sub, mul/div, mod, mod_inv; §IV-D: "the addition, subtraction, multiplication, and
// division of two multi-precision integer arrays", "mod computes the remainder of two
// multi-precision integer arrays", "mod_inv computes the modular inverse of two multiprecision
// integer arrays, used to generate key pair ... of RSA and Paillier").
//
// Batches of unsigned integers of `words` 32-bit limbs (1 <= words <= 256), element i at
// a + i * words.  Each element is held by a group of T lanes of one warp, 8 limbs per lane, in the
// smallest frame F in {32, 64, 128, 256} limbs >= words (T = F / 8), with the carry-lookahead
// group helpers of flb_bn.cuh.  Every loop has a trip count fixed by F, so the groups of a warp
// never diverge (the shuffles and ballots are full-warp):
//   add / sub   one group addition with ballot carry-lookahead; carry / borrow out per element;
//   mul         the full 2 words-limb product (row-scanning product, mul_full);
//   div / mod   binary restoring division over the (remainder : dividend) shift register,
//               32 F steps: r = 2 r + next bit, subtract b when r >= b, the decision is the
//               quotient bit; b = 0 gives q = 2^(32 words) - 1, r = a (every step "subtracts" 0);
//   mod_inv     x^-1 mod n.  Odd n: binary extended gcd of (x mod n, n) with the coefficients of x
//               kept mod n (halving t as t/2 or (t + n)/2), 64 F steps.  Even n (then x must be
//               odd): y = n^-1 mod x by the same routine with the odd modulus x, and
//               x^-1 mod n = (1 + n (x - y)) / x — an exact division, done as a product with
//               x^-1 mod 2^(32 F) (Newton iteration), because 1 + n (x - y) <= n x < 2^(32 F) x.
//               Not invertible (gcd(x, n) != 1, n < 2): out = 0, ok = 0.
#include "flb_core.cuh"

namespace flb {
namespace mp {

constexpr int X = 8;  // limbs per lane

// limbs [k X, k X + X) of an element with `words` limbs; rows 16-byte aligned only when words % 4 == 0
template <int T>
__device__ __forceinline__ void ld_elem(uint32_t (&r)[X], const uint32_t* base, uint32_t words, bool valid) {
  const int k = (int)(lane_id() & (T - 1));
  const uint32_t w0 = (uint32_t)(k * X);
  if (valid && w0 + X <= words && (words & 3u) == 0) {
    load_limbs<X>(r, base + w0);
  } else {
#pragma unroll
    for (int j = 0; j < X; j++) r[j] = (valid && w0 + j < words) ? __ldg(base + w0 + j) : 0u;
  }
}

// store this lane's limbs as words [off + k X, off + k X + X) of a row, clipped to [0, lim)
template <int T>
__device__ __forceinline__ void st_elem(uint32_t* base, const uint32_t (&r)[X], uint32_t off, uint32_t lim,
                                        bool aligned) {
  const int k = (int)(lane_id() & (T - 1));
  const uint32_t w0 = off + (uint32_t)(k * X);
  if (aligned && w0 + X <= lim) {
    store_limbs<X>(base + w0, r);
  } else {
#pragma unroll
    for (int j = 0; j < X; j++)
      if (w0 + j < lim) base[w0 + j] = r[j];
  }
}

// r <<= 1 over the group, `in` entering bit 0; returns the bit shifted out of the top (every lane)
template <int T>
__device__ __forceinline__ uint32_t shl1(uint32_t (&r)[X], uint32_t in) {
  const int k = (int)(lane_id() & (T - 1));
  const uint32_t top = r[X - 1] >> 31;
  uint32_t below = __shfl_up_sync(FULL, top, 1, T);
  if (k == 0) below = in;
#pragma unroll
  for (int j = X - 1; j > 0; j--) r[j] = __funnelshift_l(r[j - 1], r[j], 1);
  r[0] = (r[0] << 1) | below;
  return __shfl_sync(FULL, top, T - 1, T);
}

// r >>= 1 over the group, `in` entering the top bit
template <int T>
__device__ __forceinline__ void shr1(uint32_t (&r)[X], uint32_t in) {
  const int k = (int)(lane_id() & (T - 1));
  uint32_t above = __shfl_down_sync(FULL, r[0] & 1u, 1, T);
  if (k == T - 1) above = in;
#pragma unroll
  for (int j = 0; j < X - 1; j++) r[j] = __funnelshift_r(r[j], r[j + 1], 1);
  r[X - 1] = (r[X - 1] >> 1) | (above << 31);
}

// bit 0 of the group value (every lane)
template <int T>
__device__ __forceinline__ uint32_t low_bit(const uint32_t (&r)[X]) {
  return __shfl_sync(FULL, r[0] & 1u, 0, T);
}

template <int T>
__device__ __forceinline__ bool grp_is_zero(const uint32_t (&r)[X]) {
  const uint32_t nz = __ballot_sync(FULL, !all_zero<X>(r));
  const int base = (T == 32) ? 0 : (int)(lane_id() & ~(uint32_t)(T - 1));
  const uint32_t mask = (T == 32) ? 0xffffffffu : ((1u << T) - 1u);
  return ((nz >> base) & mask) == 0u;
}

__device__ __forceinline__ void sel(uint32_t (&d)[X], bool c, const uint32_t (&a)[X], const uint32_t (&b)[X]) {
#pragma unroll
  for (int j = 0; j < X; j++) d[j] = c ? a[j] : b[j];
}

// a <- floor(a / b), r <- a mod b (binary restoring division over the F-limb frame)
template <int T>
__device__ __forceinline__ void divmod(uint32_t (&a)[X], uint32_t (&r)[X], const uint32_t (&b)[X]) {
  const int k = (int)(lane_id() & (T - 1));
  zero_limbs<X>(r);
#pragma unroll 1
  for (int it = 0; it < 32 * X * T; it++) {
    const uint32_t abit = shl1<T>(a, 0u);
    const uint32_t ov = shl1<T>(r, abit);  // r < b before the shift, so the true 2r + bit < 2b
    uint32_t d[X];
    const uint32_t borrow = grp_sub<X, T>(d, r, b);
    const bool take = ov != 0u || borrow == 0u;
    sel(r, take, d, r);
    if (k == 0 && take) a[0] |= 1u;
  }
}

// t <- t / 2 mod M (M odd, t < M): t / 2 if t is even, else (t + M) / 2
template <int T>
__device__ __forceinline__ void half_mod(uint32_t (&t)[X], const uint32_t (&M)[X]) {
  const bool odd = low_bit<T>(t) != 0u;
  uint32_t m[X];
#pragma unroll
  for (int j = 0; j < X; j++) m[j] = odd ? M[j] : 0u;
  const uint32_t c = grp_add<X, T>(t, t, m);
  shr1<T>(t, c);
}

// d <- (a - b) mod M for a, b < M
template <int T>
__device__ __forceinline__ void sub_mod(uint32_t (&d)[X], const uint32_t (&a)[X], const uint32_t (&b)[X],
                                        const uint32_t (&M)[X]) {
  const uint32_t borrow = grp_sub<X, T>(d, a, b);
  uint32_t m[X];
#pragma unroll
  for (int j = 0; j < X; j++) m[j] = borrow ? M[j] : 0u;
  grp_add<X, T>(d, d, m);
}

// x2 <- u0^-1 mod M for odd M, u0 < M; returns true iff gcd(u0, M) = 1.  Binary extended gcd with
// the invariants x1 u0 = u, x2 u0 = v (mod M): each step halves an even one of (u, v), or replaces
// the larger of two odd ones by half their difference, so bits(u) + bits(v) falls every step and
// 64 F steps reach u = 0 with v = gcd(u0, M).
template <int T>
__device__ __forceinline__ bool inv_odd(uint32_t (&x2)[X], const uint32_t (&u0)[X], const uint32_t (&M)[X]) {
  const int k = (int)(lane_id() & (T - 1));
  uint32_t u[X], v[X], x1[X];
#pragma unroll
  for (int j = 0; j < X; j++) { u[j] = u0[j]; v[j] = M[j]; x1[j] = 0; x2[j] = 0; }
  if (k == 0) x1[0] = 1;
#pragma unroll 1
  for (int it = 0; it < 64 * X * T; it++) {
    const bool done = grp_is_zero<T>(u);
    const bool ue = low_bit<T>(u) == 0u, ve = low_bit<T>(v) == 0u;
    uint32_t d[X];
    const bool ge = grp_sub<X, T>(d, u, v) == 0u;
    const bool cu = ue || (!ve && ge);  // operate on (u, x1); else on (v, x2)
    const bool pe = cu ? ue : ve;
    uint32_t P[X], Q[X], p1[X], p2[X];
    sel(P, cu, u, v);
    sel(Q, cu, v, u);
    sel(p1, cu, x1, x2);
    sel(p2, cu, x2, x1);
    uint32_t diff[X], t[X];
    grp_sub<X, T>(diff, P, Q);
    sel(P, pe, P, diff);
    shr1<T>(P, 0u);
    sub_mod<T>(t, p1, p2, M);
    sel(p1, pe, p1, t);
    half_mod<T>(p1, M);
    if (!done) {
      if (cu) {
        sel(u, true, P, P);
        sel(x1, true, p1, p1);
      } else {
        sel(v, true, P, P);
        sel(x2, true, p1, p1);
      }
    }
  }
  // gcd = v == 1
  uint32_t one[X];
  zero_limbs<X>(one);
  if (k == 0) one[0] = 1;
  uint32_t d[X];
  grp_sub<X, T>(d, v, one);
  return grp_is_zero<T>(d);
}

struct MpArgs {
  const uint32_t* a;
  const uint32_t* b;
  uint32_t* out;   // add/sub/mul: result; div: quotient; mod_inv: inverse
  uint32_t* out2;  // div: remainder
  uint32_t* flag;  // add: carry, sub: borrow, mod_inv: ok (uint32 per element), optional
  uint32_t words;
  uint64_t count;
};

// op 0: add, 1: sub
template <int T, int OP>
__global__ void __launch_bounds__(32) k_mp_addsub(const MpArgs A) {
  const Grid<T> g;
  const bool al = (A.words & 3u) == 0;
  for (uint64_t base = g.wg0; base < A.count; base += g.G) {
    const uint64_t e = base + (g.gid - g.wg0);
    const bool valid = e < A.count;
    uint32_t a[X], b[X], r[X];
    ld_elem<T>(a, A.a + e * A.words, A.words, valid);
    ld_elem<T>(b, A.b + e * A.words, A.words, valid);
    uint32_t c = OP == 0 ? grp_add<X, T>(r, a, b) : grp_sub<X, T>(r, a, b);
    // carry / borrow out of bit 32 words (the frame may be wider than `words`)
    if (A.words < (uint32_t)(X * T)) {
      const int k = g.k;
      const uint32_t w = A.words, lane = w / X, j = w % X;
      uint32_t bitw = 0;
#pragma unroll
      for (int q = 0; q < X; q++)
        if ((uint32_t)q == j) bitw = r[q];
      // word `words` of r holds 1 (add) or 0xffffffff (sub, borrow) above the `words`-limb result
      c = __shfl_sync(FULL, bitw, lane, T) != 0u ? 1u : 0u;
      (void)k;
    }
    if (valid) {
      st_elem<T>(A.out + e * A.words, r, 0, A.words, al);
      if (A.flag && g.k == 0) A.flag[e] = c;
    }
  }
}

template <int T>
__global__ void __launch_bounds__(32) k_mp_mul(const MpArgs A) {
  const Grid<T> g;
  const uint32_t ow = 2 * A.words;
  const bool al = (ow & 3u) == 0;
  for (uint64_t base = g.wg0; base < A.count; base += g.G) {
    const uint64_t e = base + (g.gid - g.wg0);
    const bool valid = e < A.count;
    uint32_t a[X], b[X], lo[X], hi[X];
    ld_elem<T>(a, A.a + e * A.words, A.words, valid);
    ld_elem<T>(b, A.b + e * A.words, A.words, valid);
    mul_full<X, T>(lo, hi, a, b);
    if (valid) {
      st_elem<T>(A.out + e * ow, lo, 0, ow, al);
      st_elem<T>(A.out + e * ow, hi, X * T, ow, al);
    }
  }
}

template <int T>
__global__ void __launch_bounds__(32) k_mp_divmod(const MpArgs A) {
  const Grid<T> g;
  const bool al = (A.words & 3u) == 0;
  for (uint64_t base = g.wg0; base < A.count; base += g.G) {
    const uint64_t e = base + (g.gid - g.wg0);
    const bool valid = e < A.count;
    uint32_t a[X], b[X], r[X];
    ld_elem<T>(a, A.a + e * A.words, A.words, valid);
    ld_elem<T>(b, A.b + e * A.words, A.words, valid);
    divmod<T>(a, r, b);
    if (valid) {
      if (A.out) st_elem<T>(A.out + e * A.words, a, 0, A.words, al);
      if (A.out2) st_elem<T>(A.out2 + e * A.words, r, 0, A.words, al);
    }
  }
}

template <int T>
__global__ void __launch_bounds__(32) k_mp_modinv(const MpArgs A) {
  const Grid<T> g;
  const bool al = (A.words & 3u) == 0;
  const int k = g.k;
  for (uint64_t base = g.wg0; base < A.count; base += g.G) {
    const uint64_t e = base + (g.gid - g.wg0);
    const bool valid = e < A.count;
    uint32_t x[X], n[X];
    ld_elem<T>(x, A.a + e * A.words, A.words, valid);
    ld_elem<T>(n, A.b + e * A.words, A.words, valid);
    const bool n_odd = low_bit<T>(n) != 0u, x_odd = low_bit<T>(x) != 0u;
    // n >= 2
    uint32_t one[X], d[X];
    zero_limbs<X>(one);
    if (k == 0) one[0] = 1;
    const uint32_t nb = grp_sub<X, T>(d, n, one);  // (both collectives run in every group: no short circuit)
    const bool n1 = grp_is_zero<T>(d);
    const bool n_big = nb == 0u && !n1;
    // odd n: (u0, M) = (x mod n, n); even n: (n mod x, x)
    uint32_t A0[X], M[X], u0[X];
    sel(A0, n_odd, x, n);
    sel(M, n_odd, n, x);
    divmod<T>(A0, u0, M);
    uint32_t y[X];
    const bool g1 = inv_odd<T>(y, u0, M);
    // even n: z = (n (x - y) + 1) * x^-1 mod 2^(32 F), then z mod n (z <= n + 1)
    uint32_t xinv[X], t[X];
    {
      // x^-1 mod 2^(32 F) by Newton: inv <- inv (2 - x inv), doubling the correct bits
      const uint32_t x0 = __shfl_sync(FULL, x[0], 0, T);
      zero_limbs<X>(xinv);
      if (k == 0) xinv[0] = 0u - host_free_neg_inv32(x0 | 1u);
#pragma unroll 1
      for (int bits = 32; bits < 32 * X * T; bits *= 2) {
        mul_lo<X, T>(t, x, xinv);            // x inv
        uint32_t two[X];
        zero_limbs<X>(two);
        if (k == 0) two[0] = 2;
        grp_sub<X, T>(t, two, t);            // 2 - x inv (mod 2^(32 F))
        mul_lo<X, T>(xinv, xinv, t);
      }
    }
    uint32_t z[X];
    grp_sub<X, T>(t, x, y);
    mul_lo<X, T>(z, n, t);
    grp_add_small<X, T>(z, 1u);
    mul_lo<X, T>(z, z, xinv);
    grp_cond_sub<X, T>(z, n, 0u);
    const bool ok = n_big && g1 && (n_odd || x_odd);
    uint32_t res[X];
    sel(res, n_odd, y, z);
#pragma unroll
    for (int j = 0; j < X; j++) res[j] = ok ? res[j] : 0u;
    if (valid) {
      st_elem<T>(A.out + e * A.words, res, 0, A.words, al);
      if (A.flag && k == 0) A.flag[e] = ok ? 1u : 0u;
    }
  }
}

template <int T, typename K>
int launch(K kernel, const MpArgs& A, cudaStream_t st) {
  int grid;
  int rc = grid_for<T>(kernel, A.count, &grid);
  if (rc) return rc;
  kernel<<<grid, kBlock, 0, st>>>(A);
  FLB_LAUNCH_CHECK();
  return FLB_OK;
}

// op: 0 add, 1 sub, 2 mul, 3 divmod, 4 mod_inv
template <int T>
int run(int op, const MpArgs& A, cudaStream_t st) {
  switch (op) {
    case 0: return launch<T>(k_mp_addsub<T, 0>, A, st);
    case 1: return launch<T>(k_mp_addsub<T, 1>, A, st);
    case 2: return launch<T>(k_mp_mul<T>, A, st);
    case 3: return launch<T>(k_mp_divmod<T>, A, st);
    default: return launch<T>(k_mp_modinv<T>, A, st);
  }
}

int dispatch(int op, const MpArgs& A, void* stream) {
  if (A.words == 0 || A.words > 256) return fail(FLB_EINVAL, "words must be in [1, 256]");
  if (A.count == 0) return FLB_OK;
  cudaStream_t st = (cudaStream_t)stream;
  if (A.words <= 32) return run<4>(op, A, st);
  if (A.words <= 64) return run<8>(op, A, st);
  if (A.words <= 128) return run<16>(op, A, st);
  return run<32>(op, A, st);
}

}  // namespace mp
}  // namespace flb

extern "C" {

int flb_mp_add(const uint32_t* a, const uint32_t* b, uint32_t* out, uint32_t* carry, uint32_t words, size_t count,
               void* stream) {
  if (!a || !b || !out) return fail(FLB_EINVAL, "null pointer");
  return flb::mp::dispatch(0, flb::mp::MpArgs{a, b, out, nullptr, carry, words, count}, stream);
}

int flb_mp_sub(const uint32_t* a, const uint32_t* b, uint32_t* out, uint32_t* borrow, uint32_t words, size_t count,
               void* stream) {
  if (!a || !b || !out) return fail(FLB_EINVAL, "null pointer");
  return flb::mp::dispatch(1, flb::mp::MpArgs{a, b, out, nullptr, borrow, words, count}, stream);
}

int flb_mp_mul(const uint32_t* a, const uint32_t* b, uint32_t* out, uint32_t words, size_t count, void* stream) {
  if (!a || !b || !out) return fail(FLB_EINVAL, "null pointer");
  return flb::mp::dispatch(2, flb::mp::MpArgs{a, b, out, nullptr, nullptr, words, count}, stream);
}

int flb_mp_divmod(const uint32_t* a, const uint32_t* b, uint32_t* q, uint32_t* r, uint32_t words, size_t count,
                  void* stream) {
  if (!a || !b || (!q && !r)) return fail(FLB_EINVAL, "null pointer");
  return flb::mp::dispatch(3, flb::mp::MpArgs{a, b, q, r, nullptr, words, count}, stream);
}

int flb_mp_mod(const uint32_t* x, const uint32_t* n, uint32_t* r, uint32_t words, size_t count, void* stream) {
  if (!x || !n || !r) return fail(FLB_EINVAL, "null pointer");
  return flb::mp::dispatch(3, flb::mp::MpArgs{x, n, nullptr, r, nullptr, words, count}, stream);
}

int flb_mp_mod_inv(const uint32_t* x, const uint32_t* n, uint32_t* out, uint32_t* ok, uint32_t words, size_t count,
                   void* stream) {
  if (!x || !n || !out) return fail(FLB_EINVAL, "null pointer");
  return flb::mp::dispatch(4, flb::mp::MpArgs{x, n, out, nullptr, ok, words, count}, stream);
}

}  // extern "C"
