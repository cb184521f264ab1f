// host_bn.hpp — host-side multi-precision helpers for key setup (layer L3), no GMP.
//
// Used once per key (not on the timed path): products n = p*q, n^2, p^2, q^2; Montgomery
// constants (§III-B: "N' can be reused for all Montgomery multiplications, and
// thus, it is pre-computed"); R^k mod N by modular doubling (no long division, SURVEY §7 "host
// bignum without GMP"); inverses by Fermat through a host CIOS Montgomery exponentiation; and
// Miller–Rabin key generation.  Little-endian 32-bit limbs.
#pragma once
#include <cstdint>
#include <cstring>
#include <stdexcept>
#include <vector>

namespace flb {
namespace host {

using Limbs = std::vector<uint32_t>;

inline Limbs resized(const Limbs& a, size_t w) {
  Limbs r(w, 0);
  for (size_t i = 0; i < a.size() && i < w; i++) r[i] = a[i];
  for (size_t i = w; i < a.size(); i++)
    if (a[i]) throw std::runtime_error("resized: value does not fit");
  return r;
}

inline size_t bits(const Limbs& a) {
  for (size_t i = a.size(); i-- > 0;)
    if (a[i]) return 32 * i + (32 - __builtin_clz(a[i]));
  return 0;
}

inline bool is_zero(const Limbs& a) {
  for (uint32_t w : a)
    if (w) return false;
  return true;
}

inline bool bit(const Limbs& a, size_t i) { return (i / 32 < a.size()) && ((a[i / 32] >> (i % 32)) & 1u); }

// compare equal-length (or not) values
inline int cmp(const Limbs& a, const Limbs& b) {
  size_t w = a.size() > b.size() ? a.size() : b.size();
  for (size_t i = w; i-- > 0;) {
    uint32_t x = i < a.size() ? a[i] : 0, y = i < b.size() ? b[i] : 0;
    if (x != y) return x < y ? -1 : 1;
  }
  return 0;
}

// a -= b (a >= b), sizes: b.size() <= a.size()
inline void sub_in(Limbs& a, const Limbs& b) {
  uint64_t br = 0;
  for (size_t i = 0; i < a.size(); i++) {
    uint64_t d = (uint64_t)a[i] - (i < b.size() ? b[i] : 0) - br;
    a[i] = (uint32_t)d;
    br = (d >> 63) & 1;
  }
  if (br) throw std::runtime_error("sub_in: negative");
}

// a += b, returns carry
inline uint32_t add_in(Limbs& a, const Limbs& b) {
  uint64_t c = 0;
  for (size_t i = 0; i < a.size(); i++) {
    c += (uint64_t)a[i] + (i < b.size() ? b[i] : 0);
    a[i] = (uint32_t)c;
    c >>= 32;
  }
  return (uint32_t)c;
}

inline Limbs mul(const Limbs& a, const Limbs& b) {
  Limbs r(a.size() + b.size(), 0);
  for (size_t i = 0; i < a.size(); i++) {
    uint64_t c = 0;
    for (size_t j = 0; j < b.size(); j++) {
      c += (uint64_t)a[i] * b[j] + r[i + j];
      r[i + j] = (uint32_t)c;
      c >>= 32;
    }
    r[i + b.size()] = (uint32_t)c;
  }
  return r;
}

// x = 2x mod N for 0 <= x < N (same width as N)
inline void dbl_mod(Limbs& x, const Limbs& N) {
  uint32_t top = 0;
  for (size_t i = 0; i < x.size(); i++) {
    uint32_t nt = x[i] >> 31;
    x[i] = (x[i] << 1) | top;
    top = nt;
  }
  if (top || cmp(x, N) >= 0) {
    // x - N with the implicit top bit
    uint64_t br = 0;
    for (size_t i = 0; i < x.size(); i++) {
      uint64_t d = (uint64_t)x[i] - N[i] - br;
      x[i] = (uint32_t)d;
      br = (d >> 63) & 1;
    }
  }
}

// 2^e mod N (N odd or not; N > 1), width = N.size()
inline Limbs pow2_mod(size_t e, const Limbs& N) {
  Limbs x(N.size(), 0);
  x[0] = 1;
  if (cmp(x, N) >= 0) x[0] = 0;
  for (size_t i = 0; i < e; i++) dbl_mod(x, N);
  return x;
}

// a mod N for arbitrary-width a, by binary long division from the top bit (once per key).
inline Limbs mod(const Limbs& a, const Limbs& N) {
  Limbs r(N.size(), 0);
  for (size_t i = bits(a); i-- > 0;) {
    dbl_mod(r, N);
    if (bit(a, i)) {
      Limbs one(N.size(), 0);
      one[0] = 1;
      uint32_t c = add_in(r, one);
      if (c || cmp(r, N) >= 0) sub_in(r, N);  // r < N before, +1 keeps r <= N
    }
  }
  return r;
}

// -n0^-1 mod 2^32 (Newton iteration; n0 odd)
inline uint32_t neg_inv32(uint32_t n0) {
  uint32_t x = n0;  // correct to 3 bits
  for (int i = 0; i < 5; i++) x *= 2u - n0 * x;
  return (uint32_t)(0u - x);
}

// P^-1 mod 2^(32*w) (P odd), Newton doubling the precision each round
inline Limbs inv_mod_2k(const Limbs& P, size_t w) {
  Limbs Pw = resized(Limbs(P.begin(), P.begin() + (P.size() < w ? P.size() : w)), w);
  Limbs x(w, 0);
  x[0] = 0u - neg_inv32(Pw[0]);  // P0^-1 mod 2^32
  for (size_t prec = 1; prec < w; prec *= 2) {
    // x = x * (2 - P x) mod 2^(32w)
    const Limbs full = mul(Pw, x);
    Limbs px(full.begin(), full.begin() + w);
    Limbs two(w, 0);
    two[0] = 2;
    // t = 2 - px mod 2^(32w)
    Limbs t(w);
    uint64_t br = 0;
    for (size_t i = 0; i < w; i++) {
      uint64_t d = (uint64_t)two[i] - px[i] - br;
      t[i] = (uint32_t)d;
      br = (d >> 63) & 1;
    }
    Limbs xt = mul(x, t);
    x.assign(xt.begin(), xt.begin() + w);
  }
  return x;
}

// host CIOS Montgomery product a*b*R^-1 mod N, R = 2^(32*N.size()); a, b < N
inline Limbs mont(const Limbs& a, const Limbs& b, const Limbs& N, uint32_t n0inv) {
  const size_t s = N.size();
  std::vector<uint64_t> t(s + 2, 0);
  for (size_t i = 0; i < s; i++) {
    uint64_t c = 0;
    for (size_t j = 0; j < s; j++) {
      uint64_t v = t[j] + (uint64_t)a[j] * b[i] + c;
      t[j] = (uint32_t)v;
      c = v >> 32;
    }
    uint64_t v = t[s] + c;
    t[s] = (uint32_t)v;
    t[s + 1] = v >> 32;
    uint32_t m = (uint32_t)t[0] * n0inv;
    v = t[0] + (uint64_t)m * N[0];
    c = v >> 32;
    for (size_t j = 1; j < s; j++) {
      v = t[j] + (uint64_t)m * N[j] + c;
      t[j - 1] = (uint32_t)v;
      c = v >> 32;
    }
    v = t[s] + c;
    t[s - 1] = (uint32_t)v;
    t[s] = t[s + 1] + (v >> 32);
  }
  Limbs r(s);
  for (size_t j = 0; j < s; j++) r[j] = (uint32_t)t[j];
  if (t[s] || cmp(r, N) >= 0) {
    uint64_t br = 0;
    for (size_t j = 0; j < s; j++) {
      uint64_t d = (uint64_t)r[j] - N[j] - br;
      r[j] = (uint32_t)d;
      br = (d >> 63) & 1;
    }
  }
  return r;
}

struct MontCtx {
  Limbs N;
  uint32_t n0inv;
  Limbs R1, R2;  // R mod N, R^2 mod N
  explicit MontCtx(const Limbs& n) : N(n) {
    if (!(N[0] & 1)) throw std::runtime_error("MontCtx: even modulus");
    n0inv = neg_inv32(N[0]);
    R1 = pow2_mod(32 * N.size(), N);
    R2 = pow2_mod(64 * N.size(), N);
  }
  Limbs to(const Limbs& a) const { return mont(resized(a, N.size()), R2, N, n0inv); }
  Limbs from(const Limbs& a) const {
    Limbs one(N.size(), 0);
    one[0] = 1;
    return mont(a, one, N, n0inv);
  }
  Limbs mulmod(const Limbs& a, const Limbs& b) const { return mont(to(a), resized(b, N.size()), N, n0inv); }
  // base^e mod N (base < N), left-to-right binary
  Limbs pow(const Limbs& base, const Limbs& e) const {
    Limbs x = to(base), acc = R1;
    for (size_t i = bits(e); i-- > 0;) {
      acc = mont(acc, acc, N, n0inv);
      if (bit(e, i)) acc = mont(acc, x, N, n0inv);
    }
    return from(acc);
  }
};

// a^-1 mod P for prime P (Fermat: a^(P-2))
inline Limbs inv_mod_prime(const Limbs& a, const Limbs& P) {
  MontCtx C(P);
  Limbs e = P;
  Limbs two(P.size(), 0);
  two[0] = 2;
  sub_in(e, two);
  return C.pow(mod(a, P), e);
}

// ----------------------------------------------------------------------------- key generation
struct Xoshiro256 {
  uint64_t s[4];
  explicit Xoshiro256(uint64_t seed) {
    for (int i = 0; i < 4; i++) {  // splitmix64
      seed += 0x9E3779B97F4A7C15ull;
      uint64_t z = seed;
      z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
      z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
      s[i] = z ^ (z >> 31);
    }
  }
  static uint64_t rotl(uint64_t x, int k) { return (x << k) | (x >> (64 - k)); }
  uint64_t next() {
    const uint64_t r = rotl(s[1] * 5, 7) * 9, t = s[1] << 17;
    s[2] ^= s[0]; s[3] ^= s[1]; s[1] ^= s[2]; s[0] ^= s[3];
    s[2] ^= t; s[3] = rotl(s[3], 45);
    return r;
  }
  uint32_t next32() { return (uint32_t)(next() >> 32); }
};

inline uint32_t mod_small(const Limbs& a, uint32_t d) {
  uint64_t r = 0;
  for (size_t i = a.size(); i-- > 0;) r = ((r << 32) | a[i]) % d;
  return (uint32_t)r;
}

// a * m + add (m, add < 2^32), width grows by one word
inline Limbs mul_small(const Limbs& a, uint32_t m, uint32_t add = 0) {
  Limbs r(a.size() + 1, 0);
  uint64_t c = add;
  for (size_t i = 0; i < a.size(); i++) {
    c += (uint64_t)a[i] * m;
    r[i] = (uint32_t)c;
    c >>= 32;
  }
  r[a.size()] = (uint32_t)c;
  return r;
}

// a / d (exact or floor), d < 2^32
inline Limbs div_small(const Limbs& a, uint32_t d) {
  Limbs q(a.size(), 0);
  uint64_t r = 0;
  for (size_t i = a.size(); i-- > 0;) {
    const uint64_t cur = (r << 32) | a[i];
    q[i] = (uint32_t)(cur / d);
    r = cur % d;
  }
  return q;
}

inline const std::vector<uint32_t>& small_primes() {
  static std::vector<uint32_t> ps = [] {
    std::vector<uint32_t> v;
    for (uint32_t x = 3; x < 4000; x += 2) {
      bool pr = true;
      for (uint32_t d = 3; d * d <= x; d += 2)
        if (x % d == 0) { pr = false; break; }
      if (pr) v.push_back(x);
    }
    return v;
  }();
  return ps;
}

// Miller–Rabin with `rounds` random bases
inline bool probable_prime(const Limbs& P, Xoshiro256& rng, int rounds) {
  if (bits(P) <= 32) {
    uint64_t x = P[0];
    if (x < 2) return false;
    for (uint64_t d = 2; d * d <= x; d++)
      if (x % d == 0) return false;
    return true;
  }
  if (!(P[0] & 1)) return false;
  for (uint32_t sp : small_primes())
    if (mod_small(P, sp) == 0) return false;
  MontCtx C(P);
  Limbs pm1 = P;
  Limbs one(P.size(), 0);
  one[0] = 1;
  sub_in(pm1, one);
  size_t s = 0;
  while (!bit(pm1, s)) s++;
  Limbs d(P.size(), 0);  // d = (P-1) >> s
  for (size_t i = 0; i + s < 32 * P.size(); i++)
    if (bit(pm1, i + s)) d[i / 32] |= 1u << (i % 32);
  const Limbs mont_one = C.R1, mont_m1 = C.to(pm1);
  for (int r = 0; r < rounds; r++) {
    Limbs a(P.size(), 0);
    do {
      for (auto& w : a) w = rng.next32();
      a = mod(a, P);
    } while (bits(a) < 2 || cmp(a, pm1) >= 0);
    Limbs y = C.to(C.pow(a, d));
    if (y == mont_one || y == mont_m1) continue;
    bool ok = false;
    for (size_t i = 1; i < s; i++) {
      y = mont(y, y, C.N, C.n0inv);
      if (y == mont_m1) { ok = true; break; }
    }
    if (!ok) return false;
  }
  return true;
}

inline Limbs random_prime(size_t nbits, Xoshiro256& rng) {
  const size_t w = (nbits + 31) / 32;
  for (;;) {
    Limbs c(w, 0);
    for (auto& x : c) x = rng.next32();
    const size_t top = nbits - 1;
    if (nbits % 32) c[w - 1] &= (1u << (nbits % 32)) - 1;
    c[top / 32] |= 1u << (top % 32);
    c[(top - 1) / 32] |= 1u << ((top - 1) % 32);
    c[0] |= 1u;
    if (probable_prime(c, rng, 40)) return c;
  }
}

// ----------------------------------------------------------------------------- window schedules
// Left-to-right sliding window over odd powers ("sliding window exponential method"),
// flattened into ops: op = squarings (low 16 bits) | (table index + 1) << 16; op[0] = (0, first
// window) initialises the accumulator.  Table entry i holds base^(2i+1).
struct Schedule {
  std::vector<uint32_t> ops;
  int width = 1;
  int table = 1;
  long mults = 0;  // Montgomery multiplications incl. table (cost model)
};

inline Schedule sliding_schedule(const Limbs& e, int w) {
  Schedule S;
  S.width = w;
  S.table = 1 << (w - 1);
  long cost = (S.table > 1) ? S.table : 0;  // one squaring + table-1 products
  long i = (long)bits(e) - 1;
  if (i < 0) throw std::runtime_error("sliding_schedule: zero exponent");
  bool first = true;
  uint32_t pending_sq = 0;
  while (i >= 0) {
    if (!bit(e, i)) {
      pending_sq++;
      i--;
      continue;
    }
    long j = i - w + 1;
    if (j < 0) j = 0;
    while (!bit(e, j)) j++;
    uint32_t val = 0;
    for (long t = i; t >= j; t--) val = (val << 1) | (bit(e, t) ? 1u : 0u);
    const uint32_t len = (uint32_t)(i - j + 1);
    if (first) {
      S.ops.push_back((uint32_t)((val >> 1) + 1) << 16);
      first = false;
    } else {
      pending_sq += len;
      while (pending_sq > 0xffff) { S.ops.push_back(0xffff); cost += 0xffff; pending_sq -= 0xffff; }
      S.ops.push_back(pending_sq | ((uint32_t)((val >> 1) + 1) << 16));
      cost += pending_sq + 1;
    }
    pending_sq = 0;
    i = j - 1;
  }
  if (pending_sq) {
    while (pending_sq > 0xffff) { S.ops.push_back(0xffff); cost += 0xffff; pending_sq -= 0xffff; }
    S.ops.push_back(pending_sq);
    cost += pending_sq;
  }
  S.mults = cost;
  return S;
}

inline Schedule best_schedule(const Limbs& e, int max_w = 7) {
  Schedule best = sliding_schedule(e, 1);
  for (int w = 2; w <= max_w; w++) {
    Schedule s = sliding_schedule(e, w);
    if (s.mults < best.mults) best = s;
  }
  return best;
}

}  // namespace host
}  // namespace flb
