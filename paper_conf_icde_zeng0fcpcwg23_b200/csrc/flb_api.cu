// flb_api.cu — the C ABI (include/flb_paillier.h): key objects, constant derivation, launch
// configuration and dispatch by key frame (layer L3).
#include "flb_core.cuh"

using flb::host::Limbs;
namespace H = flb::host;
using namespace flb_rt;

namespace flb {
void set_last_error(const std::string& msg) { g_err = msg; }
void set_half_units(bool on) { flb_rt::tl_half_units = on; }
}  // namespace flb

namespace {

// Tensor-core Montgomery operands (flb_tc.cuh) for modulus N in an S-word frame, appended to blob:
// extended Toeplitz K-slices Ext[r][kk] = V_(r - KB - kk) (bytes, zero outside [0, KB)) of
// V = N' = -N^-1 mod R (2 KB rows) and V = N (3 KB rows), 32 bytes per row, in the K-major
// core-matrix layout the MMA descriptors describe (KB = 4 S).
void tc_operands(Blob& blob, const Limbs& N, uint32_t S, size_t* e1, size_t* e2) {
  auto bytes_of = [](const Limbs& v, size_t nbytes) {
    std::vector<uint8_t> b(nbytes, 0);
    for (size_t i = 0; i < nbytes && i / 4 < v.size(); i++) b[i] = (uint8_t)(v[i / 4] >> (8 * (i % 4)));
    return b;
  };
  auto ext = [&](const std::vector<uint8_t>& vb, uint32_t KB, uint32_t rows) {
    std::vector<uint8_t> m((size_t)rows * 32, 0);
    for (uint32_t r = 0; r < rows; r++)
      for (uint32_t kk = 0; kk < 32; kk++) {
        const int64_t d = (int64_t)r - KB - kk;
        if (d >= 0 && d < (int64_t)KB) m[flb::tc::cm_off(r, kk, 2)] = vb[d];
      }
    std::vector<uint32_t> w(m.size() / 4, 0);
    for (size_t i = 0; i < m.size(); i++) w[i / 4] |= (uint32_t)m[i] << (8 * (i % 4));
    return blob.put_raw(w);
  };
  const uint32_t KB = 4 * S;
  const Limbs Nf = H::resized(N, S);
  Limbs np = H::resized(H::inv_mod_2k(Nf, S), S);  // N' = R - N^-1 (two's complement)
  uint64_t cy = 1;
  for (auto& w : np) { cy += (uint32_t)~w; w = (uint32_t)cy; cy >>= 32; }
  *e1 = ext(bytes_of(np, KB), KB, 2 * KB);
  *e2 = ext(bytes_of(Nf, KB), KB, 3 * KB);
}

// largest sliding window of the key's exponent schedules; FLB_WMAX (1..7, read at key
// import) is a measurement knob for the window-table footprint
static int sched_wmax() {
  static const int w = [] {
    const char* e = getenv("FLB_WMAX");
    const int v = e ? atoi(e) : 7;
    return v < 1 ? 1 : v > 7 ? 7 : v;
  }();
  return w;
}

flb_pub* make_pub(const Limbs& n_in) {
  auto* K = new flb_pub();
  K->nbits = (uint32_t)H::bits(n_in);
  K->frame = (uint32_t)frame_for_bits(K->nbits);
  K->s = K->frame / 16;
  K->sp = K->frame / 32;
  K->n = H::resized(n_in, K->sp);
  K->n2 = H::resized(H::mul(K->n, K->n), K->s);
  H::MontCtx C(K->n2);
  K->n2_n0inv = C.n0inv;
  K->enc = H::best_schedule(K->n, sched_wmax());
  K->o_n2 = K->blob.put(K->n2, K->s);
  K->o_n = K->blob.put(K->n, K->sp);
  K->o_R2 = K->blob.put(C.R2, K->s);
  K->o_R1 = K->blob.put(C.R1, K->s);
  K->o_nR = K->blob.put(C.to(K->n), K->s);
  // R^L mod n^2 for L = 0..kReduceChunk
  std::vector<uint32_t> rl;
  Limbs cur(K->s, 0);
  cur[0] = 1;
  cur = H::mod(cur, K->n2);
  for (int L = 0; L <= kReduceChunk; L++) {
    rl.insert(rl.end(), cur.begin(), cur.end());
    cur = H::mont(cur, C.R2, K->n2, C.n0inv);  // * R
  }
  K->o_RL = K->blob.put_raw(rl);
  K->o_sched = K->blob.put_raw(K->enc.ops);
  K->o_one = K->blob.put_raw(std::vector<uint32_t>{1u, 0u, 0u, 0u});
  // public-key encryption on the tensor cores (n^2 of 64 or 128 words; k_tc_exp starts from a table
  // entry and needs at least one more schedule op)
  if ((K->s == 64 || K->s == 128) && K->enc.ops.size() >= 2) {
    tc_operands(K->blob, K->n2, K->s, &K->o_tcE1, &K->o_tcE2);
    K->tc = true;
  }
  return K;
}

flb_priv* make_priv(const Limbs& p_in, const Limbs& q_in) {
  Limbs p = p_in, q = q_in;
  if (H::cmp(p, q) < 0) std::swap(p, q);
  const Limbs n = H::mul(p, q);
  auto* V = new flb_priv();
  V->pub = make_pub(n);
  const uint32_t sp = V->pub->sp;
  V->p = H::resized(p, sp);
  V->q = H::resized(q, sp);
  Limbs one(sp, 0);
  one[0] = 1;
  for (int i = 0; i < 2; i++) {
    auto& R = V->pr[i];
    const Limbs& P = i == 0 ? V->p : V->q;
    const Limbs& Q = i == 0 ? V->q : V->p;
    R.P = P;
    R.P2 = H::resized(H::mul(P, P), sp);
    H::MontCtx C2(R.P2), C1(R.P);
    R.P2_n0inv = C2.n0inv;
    R.P_n0inv = C1.n0inv;
    Limbs pm1 = P;
    H::sub_in(pm1, one);
    R.sched = H::best_schedule(pm1, sched_wmax());
    // h_P = (-Q)^-1 mod P
    Limbs negQ = P;
    H::sub_in(negQ, H::mod(Q, P));
    const Limbs h = H::inv_mod_prime(negQ, P);
    R.o_P2 = V->blob.put(R.P2, sp);
    R.o_R2 = V->blob.put(C2.R2, sp);
    R.o_R3 = V->blob.put(H::mont(C2.R2, C2.R2, R.P2, C2.n0inv) /* R^3 mod P^2 */, sp);
    R.o_P = V->blob.put(P, sp);
    R.o_Pinv = V->blob.put(H::inv_mod_2k(P, sp), sp);
    R.o_hR = V->blob.put(C1.to(h), sp);
    R.o_sched = V->blob.put_raw(R.sched.ops);
    R.o_nR = V->blob.put(C2.to(H::mod(V->pub->n, R.P2)), sp);
  }
  {
    // (q^2)^-1 mod p^2 by Euler: a^(phi(p^2) - 1), phi(p^2) = p (p - 1)
    H::MontCtx Cp2(V->pr[0].P2);
    Limbs phi = H::resized(H::mul(V->p, [&] { Limbs t = V->p; H::sub_in(t, one); return t; }()), 2 * sp);
    Limbs e = phi;
    Limbs one2(e.size(), 0);
    one2[0] = 1;
    H::sub_in(e, one2);
    const Limbs q2inv = Cp2.pow(H::mod(V->pr[1].P2, V->pr[0].P2), e);
    V->o_q2invR = V->blob.put(Cp2.to(q2inv), sp);
    V->o_enc_sched = V->blob.put_raw(V->pub->enc.ops);
  }
  {
    // v2 half frame: the smallest supported frame holding p; used only when it is below sp
    uint32_t Hf = 0;
    const uint32_t pw = (uint32_t)((H::bits(V->p) + 31) / 32);
    for (uint32_t f : {32u, 64u, 96u, 128u})
      if (pw <= f) { Hf = f; break; }
    if (Hf && Hf < sp) {
      V->H = Hf;
      for (int i = 0; i < 2; i++) {
        const Limbs P = H::resized(i == 0 ? V->p : V->q, Hf);
        H::MontCtx C(P);
        V->half[i].n0inv = C.n0inv;
        V->half[i].o_P = V->blob.put(P, Hf);
        V->half[i].o_R2 = V->blob.put(C.R2, Hf);
        V->half[i].o_R3 = V->blob.put(H::mont(C.R2, C.R2, P, C.n0inv), Hf);
      }
      V->sched_p = H::best_schedule(V->p, sched_wmax());
      V->sched_q = H::best_schedule(V->q, sched_wmax());
      V->o_sched_p = V->blob.put_raw(V->sched_p.ops);
      V->o_sched_q = V->blob.put_raw(V->sched_q.ops);
    }
  }
  // tensor-core Montgomery operands (flb_tc.cuh) for the P^2 moduli when sp is 32, 64, 96 or 128
  // (decryption, key-holder encryption stage 2) and for the half-frame P moduli when H is 32 or 64
  // (key-holder encryption stage 1)
  {
    auto operands = [&](const Limbs& N, uint32_t S, size_t* e1, size_t* e2) { tc_operands(V->blob, N, S, e1, e2); };
    // (k_tc_exp starts from a table entry and needs at least one more schedule op: toy keys with
    // one-window exponents stay on the CIOS kernels)
    if ((sp == 32 || sp == 64 || sp == 96 || sp == 128) && V->pr[0].sched.ops.size() >= 2 &&
        V->pr[1].sched.ops.size() >= 2) {
      for (int i = 0; i < 2; i++) operands(V->pr[i].P2, sp, &V->pr[i].o_tcE1, &V->pr[i].o_tcE2);
      V->tc = true;
    }
    if (V->H == 32 || V->H == 64) {
      for (int i = 0; i < 2; i++) operands(i == 0 ? V->p : V->q, V->H, &V->half[i].o_tcE1, &V->half[i].o_tcE2);
      V->tc_half = true;
    }
    V->o_one = V->blob.put_raw(std::vector<uint32_t>{1u, 0u, 0u, 0u});
  }
  // CRT recombination constants
  H::MontCtx Cn(V->pub->n), Cp(V->p);
  V->n_n0inv = Cn.n0inv;
  V->o_n = V->blob.put(V->pub->n, sp);
  V->o_qR_n = V->blob.put(Cn.to(V->q), sp);
  V->o_qinvR_p = V->blob.put(Cp.to(H::inv_mod_prime(V->q, V->p)), sp);
  return V;
}

flb_mod* make_mod(const Limbs& n_in, uint32_t S) {
  auto* M = new flb_mod();
  flb_pub& K = M->core;
  K.nbits = (uint32_t)H::bits(n_in);
  K.s = S;
  K.sp = S / 2;
  K.frame = 16 * S;  // the dispatch key: S limbs is the "n^2" frame of a 16*S... i.e. 1024 <-> 64 limbs
  K.n2 = H::resized(n_in, S);
  H::MontCtx C(K.n2);
  K.n2_n0inv = C.n0inv;
  K.o_n2 = K.blob.put(K.n2, S);
  K.o_R2 = K.blob.put(C.R2, S);
  K.o_R1 = K.blob.put(C.R1, S);
  return M;
}
}  // namespace

// ----------------------------------------------------------------------------- dispatch macros
// Limb split per frame: X limbs per lane, T lanes per big integer.  FLB_LIMBS=8 selects the
// narrow split (tuning experiments); the default is the wide split.
static int limbs_per_lane() {
  static int v = [] {
    const char* e = getenv("FLB_LIMBS");
    return (e && atoi(e) == 8) ? 8 : 16;
  }();
  return v;
}
#define FLB_DISPATCH_ENC(frame, FN, ...)                                           \
  do {                                                                            \
    const bool nar = limbs_per_lane() == 8;                                       \
    switch (frame) {                                                              \
      case 512: return FN<16, 2>(__VA_ARGS__);  /* generic moduli of <= 32 limbs */ \
      case 1024: return nar ? FN<8, 8>(__VA_ARGS__) : FN<16, 4>(__VA_ARGS__);     \
      case 1536: return FN<12, 8>(__VA_ARGS__); /* generic moduli of <= 96 limbs */ \
      case 2048: return nar ? FN<8, 16>(__VA_ARGS__) : FN<16, 8>(__VA_ARGS__);    \
      case 3072: return FN<12, 16>(__VA_ARGS__);                                  \
      case 4096: return nar ? FN<8, 32>(__VA_ARGS__) : FN<16, 16>(__VA_ARGS__);   \
      default: return fail(FLB_EUNSUPPORTED, "unsupported key frame");            \
    }                                                                             \
  } while (0)
#define FLB_DISPATCH_DEC(frame, FN, ...)                                           \
  do {                                                                            \
    const bool nar = limbs_per_lane() == 8;                                       \
    switch (frame) {                                                              \
      case 1024: return nar ? FN<8, 4>(__VA_ARGS__) : FN<16, 2>(__VA_ARGS__);     \
      case 2048: return nar ? FN<8, 8>(__VA_ARGS__) : FN<16, 4>(__VA_ARGS__);     \
      case 3072: return FN<12, 8>(__VA_ARGS__);                                   \
      case 4096: return nar ? FN<8, 16>(__VA_ARGS__) : FN<16, 8>(__VA_ARGS__);    \
      default: return fail(FLB_EUNSUPPORTED, "unsupported key frame");            \
    }                                                                             \
  } while (0)

namespace {
template <int X, int T>
int run_add_plain(const flb_pub* K, const uint32_t* dev, const uint32_t* a, const uint32_t* b, uint32_t* out,
                  size_t count, cudaStream_t st) {
  return run_add<X, T, false>(K, dev, a, b, out, count, st);
}
template <int X, int T>
int run_mont_dbg(const flb_pub* K, const uint32_t* dev, const uint32_t* a, const uint32_t* b, uint32_t* out,
                 size_t count, cudaStream_t st) {
  return run_add<X, T, true>(K, dev, a, b, out, count, st);
}
}  // namespace

extern "C" {

const char* flb_last_error(void) { return g_err.c_str(); }

static uint64_t sched_mults(const H::Schedule& S) {
  uint64_t m = (S.table > 1) ? (uint64_t)S.table : 0;  // x^2 + (table-1) products
  for (size_t i = 1; i < S.ops.size(); i++) m += (S.ops[i] & 0xffffu) + ((S.ops[i] >> 16) ? 1 : 0);
  return m;
}

static uint64_t sched_squarings(const H::Schedule& S) {
  uint64_t q = (S.table > 1) ? 1u : 0u;  // x^2 of the table
  for (size_t i = 1; i < S.ops.size(); i++) q += S.ops[i] & 0xffffu;
  return q;
}

// IMAD-pipe limb products of the tensor-core kernel (flb_tc.cuh) for `mults` S-word Montgomery
// products of which `sqr` are squarings: S^2 for the row-scan product, S (S + 1) / 2 for the block
// squaring with triangular diagonal blocks
static uint64_t tc_imad_lp(uint64_t S, uint64_t mults, uint64_t sqr) {
  return (mults - sqr) * S * S + sqr * (S * (S + 1) / 2);
}

// u8 MACs the two Toeplitz MMAs of one S-word tensor-core Montgomery product issue per element (MMA
// row): K-slices of 32 bytes, q = t N' mod R over columns [32 ks, KB), q N over [0, min(KB, 32 ks + 48))
// (flb_tc.cuh mma_toeplitz_lo / _hi)
static uint64_t tc_mma_macs(uint64_t S) {
  const uint64_t KB = 4 * S;
  uint64_t m = 0;
  for (uint64_t ks = 0; ks < KB / 32; ks++) m += 32 * (KB - 32 * ks) + 32 * std::min<uint64_t>(KB, 32 * ks + 48);
  return m;
}

int flb_op_cost(const flb_pub* K, const flb_priv* V, int op, uint64_t* mont_muls, uint64_t* limb_products) {
  if (!mont_muls || !limb_products) return fail(FLB_EINVAL, "null output");
  const flb_pub* P = K ? K : (V ? V->pub : nullptr);
  if (!P) return fail(FLB_EINVAL, "null key");
  const uint64_t s = P->s, sp = P->sp, cs = 2 * s * s + s, csp = 2 * sp * sp + sp;
  switch (op) {
    case 0: {  // encrypt: to-Montgomery, table + schedule, m n, final product
      const uint64_t mm = 1 + sched_mults(P->enc) + 2;
      *mont_muls = mm;
      *limb_products = mm * cs;
      return FLB_OK;
    }
    case 1: {  // decrypt: per prime 2 (entry) + table + schedule + 1 (exit) + 1 (h_P); mul_lo; CRT 2
      if (!V) return fail(FLB_EINVAL, "decrypt cost needs the private key");
      uint64_t mm = 2, lp = 0;
      for (int i = 0; i < 2; i++) {
        mm += 2 + sched_mults(V->pr[i].sched) + 1 + 1;
        lp += sp * sp;  // exact division (low half product)
      }
      *mont_muls = mm;
      *limb_products = mm * csp + lp;
      return FLB_OK;
    }
    case 4: {  // key-holder encryption
      if (!V) return fail(FLB_EINVAL, "key-holder cost needs the private key");
      if (V->H) {
        // v2: per prime, stage 1 at the half frame (2 entry + table + schedule(Q) + exit) and stage 2
        // at sp (entry + table + schedule(P) + m n + final); CRT 1 + plain product
        const uint64_t h = V->H, ch = 2 * h * h + h;
        const uint64_t s1 = (2 + sched_mults(V->sched_q) + 1) + (2 + sched_mults(V->sched_p) + 1);
        const uint64_t s2 = (1 + sched_mults(V->sched_p) + 2) + (1 + sched_mults(V->sched_q) + 2) + 1;
        *mont_muls = s1 + s2;
        *limb_products = s1 * ch + s2 * csp + sp * sp;
        return FLB_OK;
      }
      const uint64_t per = 1 + sched_mults(P->enc) + 2;
      *mont_muls = 2 * per + 1;
      *limb_products = (2 * per + 1) * csp + sp * sp;
      return FLB_OK;
    }
    case 5: {  // key-holder encryption, tensor-core kernels (k_tc_exp) only: stage 1 at H, stage 2 at sp.
      // Montgomery products on the tensor-core path; limb_products = the S^2 32x32-bit products of
      // t = a b on the IMAD pipe (the reduction's u8 MACs are 32 S^2 per product: 2 MMAs of KB^2)
      if (V && V->tc && !V->H && sp == 32) {
        // one stage per prime (run_encrypt_crt1_tc): 1 (entry) + table + schedule(n) + m n + final
        const uint64_t mm = 2 * (1 + sched_mults(P->enc) + 2), sq = 2 * sched_squarings(P->enc);
        *mont_muls = mm;
        *limb_products = tc_imad_lp(sp, mm, sq);
        return FLB_OK;
      }
      if (!V || !V->tc || !V->tc_half) return fail(FLB_EUNSUPPORTED, "no tensor-core key-holder path for this key");
      const uint64_t h = V->H;
      const uint64_t s1 = (2 + sched_mults(V->sched_q) + 1) + (2 + sched_mults(V->sched_p) + 1);
      const uint64_t s2 = (1 + sched_mults(V->sched_p) + 2) + (1 + sched_mults(V->sched_q) + 2);
      const uint64_t q12 = sched_squarings(V->sched_q) + sched_squarings(V->sched_p);  // same exponents
      *mont_muls = s1 + s2;
      *limb_products = tc_imad_lp(h, s1, q12) + tc_imad_lp(sp, s2, q12);
      return FLB_OK;
    }
    case 6: {  // decryption, tensor-core kernel (k_tc_exp) only: per prime 2 (entry) + table + schedule + 1
      if (!V || !V->tc) return fail(FLB_EUNSUPPORTED, "no tensor-core decryption path for this key");
      uint64_t mm = 0, sq = 0;
      for (int i = 0; i < 2; i++) {
        mm += 2 + sched_mults(V->pr[i].sched) + 1;
        sq += sched_squarings(V->pr[i].sched);
      }
      *mont_muls = mm;
      *limb_products = tc_imad_lp(sp, mm, sq);
      return FLB_OK;
    }
    case 7:    // key-holder encryption, tensor-core kernels: *limb_products = u8 MACs the MMAs issue per element
               // (triangular K-slices, tc_mma_macs)
    case 8: {  // decryption exponentiations, tensor-core kernel: likewise
      uint64_t mm, lp;
      const int rc = flb_op_cost(K, V, op - 2, &mm, &lp);
      if (rc) return rc;
      if (op == 7 && !V->H) {
        *limb_products = mm * tc_mma_macs(sp);
      } else if (op == 7) {
        const uint64_t h = V->H;
        const uint64_t s1 = (2 + sched_mults(V->sched_q) + 1) + (2 + sched_mults(V->sched_p) + 1);
        *limb_products = s1 * tc_mma_macs(h) + (mm - s1) * tc_mma_macs(sp);
      } else {
        *limb_products = mm * tc_mma_macs(sp);
      }
      *mont_muls = mm;
      return FLB_OK;
    }
    case 9:     // public-key encryption, tensor-core kernel (k_tc_exp in the n^2 frame): IMAD limb products
    case 10: {  // ... and its u8 MMA MACs
      if (!P->tc) return fail(FLB_EUNSUPPORTED, "no tensor-core public-key path for this key");
      const uint64_t mm = 1 + sched_mults(P->enc) + 2;
      *mont_muls = mm;
      *limb_products = op == 9 ? tc_imad_lp(s, mm, sched_squarings(P->enc)) : mm * tc_mma_macs(s);
      return FLB_OK;
    }
    case 2:
      *mont_muls = 2;
      *limb_products = 2 * cs;
      return FLB_OK;
    case 3:
      *mont_muls = 1;
      *limb_products = cs;
      return FLB_OK;
  }
  return fail(FLB_EINVAL, "unknown op");
}
const char* flb_version(void) { return "flb-b200 0.1 (sm_100a)"; }

int flb_keygen(uint32_t key_bits, uint64_t seed, flb_pub** pub, flb_priv** priv) {
  if (!pub || !priv) return fail(FLB_EINVAL, "null output pointer");
  if (key_bits != 1024 && key_bits != 2048 && key_bits != 3072 && key_bits != 4096)
    return fail(FLB_EINVAL, "key_bits must be 1024, 2048, 3072 or 4096");
  try {
    H::Xoshiro256 rng(seed);
    for (;;) {
      Limbs p = H::random_prime(key_bits / 2, rng), q = H::random_prime(key_bits / 2, rng);
      if (H::cmp(p, q) == 0) continue;
      Limbs n = H::mul(p, q);
      if (H::bits(n) != key_bits) continue;
      flb_priv* V = make_priv(p, q);
      *priv = V;
      *pub = make_pub(V->pub->n);
      return FLB_OK;
    }
  } catch (const std::bad_alloc&) {
    return fail(FLB_ENOMEM, "host allocation failed");
  } catch (const std::exception& ex) {
    return fail(FLB_EKEY, ex.what());
  }
}

int flb_key_from_primes(const uint32_t* p, const uint32_t* q, uint32_t prime_words, flb_pub** pub, flb_priv** priv) {
  if (!p || !q || !pub || !priv || prime_words == 0) return fail(FLB_EINVAL, "null pointer or zero size");
  try {
    Limbs P(p, p + prime_words), Q(q, q + prime_words);
    if (H::cmp(P, Q) == 0) return fail(FLB_EKEY, "p == q");
    if (!(P[0] & 1) || !(Q[0] & 1) || H::bits(P) < 2 || H::bits(Q) < 2) return fail(FLB_EKEY, "primes must be odd and >= 3");
    const Limbs n = H::mul(P, Q);
    if (H::bits(n) > 4096) return fail(FLB_EUNSUPPORTED, "bits(n) > 4096");
    H::Xoshiro256 rng(0x5eed);
    if (!H::probable_prime(P, rng, 20) || !H::probable_prime(Q, rng, 20)) return fail(FLB_EKEY, "a prime failed Miller-Rabin");
    // gcd(n, (p-1)(q-1)) = 1  <=>  p does not divide q-1 and q does not divide p-1
    Limbs one(prime_words, 0);
    one[0] = 1;
    Limbs pm1 = P, qm1 = Q;
    H::sub_in(pm1, one);
    H::sub_in(qm1, one);
    if (H::is_zero(H::mod(qm1, P)) || H::is_zero(H::mod(pm1, Q))) return fail(FLB_EKEY, "gcd(n, phi(n)) != 1");
    size_t pw = prime_words;
    while (pw > 1 && P[pw - 1] == 0 && Q[pw - 1] == 0) pw--;
    flb_priv* V = make_priv(H::resized(P, pw), H::resized(Q, pw));
    *priv = V;
    *pub = make_pub(V->pub->n);
    return FLB_OK;
  } catch (const std::bad_alloc&) {
    return fail(FLB_ENOMEM, "host allocation failed");
  } catch (const std::exception& ex) {
    return fail(FLB_EKEY, ex.what());
  }
}

int flb_key_export(const flb_priv* V, uint32_t* p, uint32_t* q, uint32_t* n) {
  if (!V) return fail(FLB_EINVAL, "null key");
  const uint32_t half = V->pub->sp / 2;
  if (p) for (uint32_t i = 0; i < half; i++) p[i] = V->p[i];
  if (q) for (uint32_t i = 0; i < half; i++) q[i] = V->q[i];
  if (n) for (uint32_t i = 0; i < V->pub->sp; i++) n[i] = V->pub->n[i];
  return FLB_OK;
}

void flb_pub_free(flb_pub* pub) { delete pub; }
void flb_priv_free(flb_priv* priv) { delete priv; }
uint32_t flb_key_bits(const flb_pub* K) { return K ? K->nbits : 0; }
uint32_t flb_pt_words(const flb_pub* K) { return K ? K->sp : 0; }
uint32_t flb_ct_words(const flb_pub* K) { return K ? K->s : 0; }
uint32_t flb_slot_capacity(const flb_pub* K, uint32_t slot_bits) {
  return (K && slot_bits) ? (K->nbits - 1) / slot_bits : 0;
}

}  // extern "C"

// ----------------------------------------------------------------------------- FLB_DEBUG_CHECKS
// With FLB_DEBUG_CHECKS=1 in the environment (read per call) the batch calls first run range-check
// kernels over their inputs (m < n, c < n^2, idx / offsets well formed, summands <= 2^pad_bits),
// wait for them and return FLB_EINVAL naming the violation; off (the default) the hot path checks
// nothing beyond the synchronous argument checks (include/flb_paillier.h).
static int dbg_grid(uint64_t n) { return (int)std::max<uint64_t>(1, std::min<uint64_t>((n + 255) / 256, 4096)); }
static bool debug_checks() {
  const char* e = getenv("FLB_DEBUG_CHECKS");
  return e && atoi(e) != 0;
}
template <typename F>
static int run_check(cudaStream_t st, const std::string& what, F launch) {
  unsigned long long* d = nullptr;
  unsigned long long h = 0;
  FLB_CK(cudaMallocAsync(&d, sizeof(h), st));
  FLB_CK(cudaMemsetAsync(d, 0, sizeof(h), st));
  launch(d);
  cudaError_t e = cudaGetLastError();
  if (e == cudaSuccess) e = cudaMemcpyAsync(&h, d, sizeof(h), cudaMemcpyDeviceToHost, st);
  cudaFreeAsync(d, st);
  if (e == cudaSuccess) e = cudaStreamSynchronize(st);
  if (e != cudaSuccess) return fail(FLB_ECUDA, std::string("FLB_DEBUG_CHECKS: ") + cudaGetErrorString(e));
  if (h) return fail(FLB_EINVAL, "FLB_DEBUG_CHECKS: " + std::to_string(h) + " " + what);
  return FLB_OK;
}
// rows x_i ([count][words], contiguous) must be < bound (device, words limbs)
static int check_below(const uint32_t* x, uint64_t count, uint32_t words, const uint32_t* bound, void* stream,
                       const char* what) {
  cudaStream_t st = (cudaStream_t)stream;
  return run_check(st, what, [&](unsigned long long* d) {
    flb::k_check_below<<<dbg_grid(count), 256, 0, st>>>(x, count, words, bound, words, d);
  });
}
static int check_segments(const int64_t* idx, size_t num_entries, size_t num_inputs, const int64_t* offsets,
                          size_t num_segments, void* stream) {
  cudaStream_t st = (cudaStream_t)stream;
  int rc = run_check(st, "malformed offsets (offsets[0] = 0, non-decreasing, offsets[S] = num_entries)",
                     [&](unsigned long long* d) {
                       flb::k_check_offsets<<<dbg_grid(num_segments + 1), 256, 0, st>>>(offsets, num_segments,
                                                                                     (int64_t)num_entries, d);
                     });
  if (rc || !idx || num_entries == 0) return rc;
  return run_check(st, "idx entries outside [0, num_inputs)", [&](unsigned long long* d) {
    flb::k_check_index<<<dbg_grid(num_entries), 256, 0, st>>>(idx, num_entries, (int64_t)num_inputs, d);
  });
}
static int pub_dev(const flb_pub* K, uint32_t** dev) { return const_cast<DevBlob&>(K->dev).get(K->blob, dev); }

extern "C" {

// tensor-core Montgomery paths (flb_tc.cuh): on when the key has the operands; FLB_TC=0 selects
// the CIOS kernels, FLB_TC=2 the tensor-core kernels at every batch size (read per call, so tests
// can compare both)
static int tc_mode() {
  const char* e = getenv("FLB_TC");
  return e ? atoi(e) : 1;
}
static bool tc_enabled() { return tc_mode() != 0; }
// Public-key encryption: a tensor-core tile is 128 elements on one CTA for the whole modexp, so a
// small batch (a few tiles on a few SMs) finishes later than the CIOS kernel spread over groups of
// T lanes: measured crossover ≈ 12 K elements at 1024 and 2048 bits (C1's 2,000 encryptions: 8.6 ms
// CIOS vs 16.5 ms on the tensor cores); below 96 elements per SM the CIOS kernel runs.
static bool tc_batch(size_t count) {
  const int mode = tc_mode();
  if (mode == 0) return false;
  if (mode == 2) return true;
  int dev = 0, sms = 148;
  if (cudaGetDevice(&dev) != cudaSuccess || cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev) != cudaSuccess) {
    (void)cudaGetLastError();
    sms = 148;
  }
  return count >= (size_t)96 * (size_t)sms;
}
// FLB_TC_DAG=0: the two key-holder stages as two k_tc_exp launches instead of one k_tc_exp_dag
static bool tc_dag_enabled() {
  const char* e = getenv("FLB_TC_DAG");
  return !(e && atoi(e) == 0);
}
static bool use_tc(const flb_priv* V) { return V->tc && tc_enabled(); }
static bool use_tc_half(const flb_priv* V) { return V->tc_half && tc_enabled(); }

int flb_encrypt(const flb_pub* K, const uint32_t* m, const uint32_t* r, uint64_t seed, uint64_t ctr0, uint32_t* c,
                size_t count, void* stream) {
  if (!K || !m || !c) return fail(FLB_EINVAL, "null pointer");
  if (count == 0) return FLB_OK;
  uint32_t* dev;
  int rc = const_cast<DevBlob&>(K->dev).get(K->blob, &dev);
  if (rc) return rc;
  if (debug_checks() && (rc = check_below(m, count, K->sp, dev + K->o_n, stream, "plaintexts m >= n"))) return rc;
  if (K->tc && tc_batch(count)) {
    if (K->s == 128) return run_encrypt_pub_tc<128>(K, dev, m, r, seed, ctr0, c, count, (cudaStream_t)stream);
    return run_encrypt_pub_tc<64>(K, dev, m, r, seed, ctr0, c, count, (cudaStream_t)stream);
  }
  FLB_DISPATCH_ENC(K->frame, run_encrypt, K, dev, m, r, seed, ctr0, c, count, (cudaStream_t)stream);
}


int flb_decrypt(const flb_priv* V, const uint32_t* c, uint32_t* m, size_t count, void* stream) {
  if (!V || !c || !m) return fail(FLB_EINVAL, "null pointer");
  if (count == 0) return FLB_OK;
  uint32_t* dev;
  int rc = const_cast<DevBlob&>(V->dev).get(V->blob, &dev);
  if (rc) return rc;
  if (debug_checks()) {
    uint32_t* pd;
    if ((rc = pub_dev(V->pub, &pd)) ||
        (rc = check_below(c, count, V->pub->s, pd + V->pub->o_n2, stream, "ciphertexts c >= n^2")))
      return rc;
  }
  if (use_tc(V)) {
    if (V->pub->sp == 128) return run_decrypt_tc<128>(V, dev, c, m, count, (cudaStream_t)stream);
    if (V->pub->sp == 96) return run_decrypt_tc<96>(V, dev, c, m, count, (cudaStream_t)stream);
    if (V->pub->sp == 64) return run_decrypt_tc<64>(V, dev, c, m, count, (cudaStream_t)stream);
    return run_decrypt_tc<32>(V, dev, c, m, count, (cudaStream_t)stream);
  }
  FLB_DISPATCH_DEC(V->pub->frame, run_decrypt, V, dev, c, m, count, (cudaStream_t)stream);
}

static int encrypt_crt_v2(const flb_priv* V, const uint32_t* dev, const uint32_t* m, const uint32_t* r, uint64_t seed,
                          uint64_t ctr0, uint32_t* c, size_t count, cudaStream_t st);

int flb_encrypt_crt(const flb_priv* V, const uint32_t* m, const uint32_t* r, uint64_t seed, uint64_t ctr0,
                    uint32_t* c, size_t count, void* stream) {
  if (!V || !m || !c) return fail(FLB_EINVAL, "null pointer");
  if (count == 0) return FLB_OK;
  uint32_t* dev;
  int rc = const_cast<DevBlob&>(V->dev).get(V->blob, &dev);
  if (rc) return rc;
  if (debug_checks()) {
    uint32_t* pd;
    if ((rc = pub_dev(V->pub, &pd)) ||
        (rc = check_below(m, count, V->pub->sp, pd + V->pub->o_n, stream, "plaintexts m >= n")))
      return rc;
  }
  if (V->H) return encrypt_crt_v2(V, dev, m, r, seed, ctr0, c, count, (cudaStream_t)stream);
  // one stage per prime (1024-bit keys): (1 + m n) r^n mod P^2 on the tensor cores for large batches
  if (V->tc && V->pub->sp == 32 && tc_batch(count))
    return run_encrypt_crt1_tc<32>(V, dev, m, r, seed, ctr0, c, count, (cudaStream_t)stream);
  FLB_DISPATCH_DEC(V->pub->frame, run_encrypt_crt, V, dev, m, r, seed, ctr0, c, count, (cudaStream_t)stream);
}

int flb_add(const flb_pub* K, const uint32_t* c1, const uint32_t* c2, uint32_t* out, size_t count, void* stream) {
  if (!K || !c1 || !c2 || !out) return fail(FLB_EINVAL, "null pointer");
  if (count == 0) return FLB_OK;
  uint32_t* dev;
  int rc = const_cast<DevBlob&>(K->dev).get(K->blob, &dev);
  if (rc) return rc;
  if (debug_checks() && ((rc = check_below(c1, count, K->s, dev + K->o_n2, stream, "c1 >= n^2")) ||
                         (rc = check_below(c2, count, K->s, dev + K->o_n2, stream, "c2 >= n^2"))))
    return rc;
  FLB_DISPATCH_ENC(K->frame, run_add_plain, K, dev, c1, c2, out, count, (cudaStream_t)stream);
}

int flb_debug_tc_product(const uint32_t* a, const uint32_t* b, uint32_t* t, uint32_t count, uint32_t words, int square,
                         void* stream) {
  if (!a || !b || !t || count > (uint32_t)flb::tc::kTileM) return fail(FLB_EINVAL, "null pointer or count > 128");
  if (words == 128) return run_tc_debug_product<128>(a, b, t, count, square, (cudaStream_t)stream);
  if (words == 96) return run_tc_debug_product<96>(a, b, t, count, square, (cudaStream_t)stream);
  if (words == 64) return run_tc_debug_product<64>(a, b, t, count, square, (cudaStream_t)stream);
  if (words == 32) return run_tc_debug_product<32>(a, b, t, count, square, (cudaStream_t)stream);
  return fail(FLB_EINVAL, "words must be 32, 64, 96 or 128");
}

int flb_debug_mont_mul(const flb_pub* K, const uint32_t* a, const uint32_t* b, uint32_t* out, size_t count,
                       void* stream) {
  if (!K || !a || !b || !out) return fail(FLB_EINVAL, "null pointer");
  if (count == 0) return FLB_OK;
  uint32_t* dev;
  int rc = const_cast<DevBlob&>(K->dev).get(K->blob, &dev);
  if (rc) return rc;
  FLB_DISPATCH_ENC(K->frame, run_mont_dbg, K, dev, a, b, out, count, (cudaStream_t)stream);
}

int flb_scalar_mul(const flb_pub* K, const uint32_t* c, const uint32_t* e, uint32_t e_words, uint32_t* out,
                   size_t count, void* stream) {
  if (!K || !c || !e || !out) return fail(FLB_EINVAL, "null pointer");
  if (e_words < 1 || e_words > 128) return fail(FLB_EINVAL, "e_words must be in [1, 128]");
  if (count == 0) return FLB_OK;
  uint32_t* dev;
  int rc = const_cast<DevBlob&>(K->dev).get(K->blob, &dev);
  if (rc) return rc;
  if (debug_checks() && (rc = check_below(c, count, K->s, dev + K->o_n2, stream, "ciphertexts c >= n^2"))) return rc;
  FLB_DISPATCH_ENC(K->frame, run_smul, K, dev, c, e, e_words, out, count, (cudaStream_t)stream);
}

int flb_reduce_segments(const flb_pub* K, const uint32_t* c, size_t num_inputs, const int64_t* idx,
                        size_t num_entries, const int64_t* offsets, size_t num_segments, size_t max_segment_len,
                        uint32_t* out, void* stream) {
  if (!K || !offsets || !out) return fail(FLB_EINVAL, "null pointer");
  if (num_entries > 0 && (!c || num_inputs == 0)) return fail(FLB_EINVAL, "null or empty input");
  if (!idx && num_entries > num_inputs) return fail(FLB_EINVAL, "without idx, num_entries must be <= num_inputs");
  if (num_segments == 0) return FLB_OK;
  uint32_t* dev;
  int rc = const_cast<DevBlob&>(K->dev).get(K->blob, &dev);
  if (rc) return rc;
  if (debug_checks() &&
      ((rc = check_segments(idx, num_entries, num_inputs, offsets, num_segments, stream)) ||
       (num_inputs && (rc = check_below(c, num_inputs, K->s, dev + K->o_n2, stream, "ciphertexts c >= n^2")))))
    return rc;
  FLB_DISPATCH_ENC(K->frame, run_reduce, K, dev, c, num_entries, idx, offsets, num_segments, max_segment_len, out,
                   (cudaStream_t)stream);
}

static int grid_1d(uint64_t n);

int flb_mod_create(const uint32_t* n, uint32_t words, flb_mod** out) {
  if (!n || !out || words == 0) return fail(FLB_EINVAL, "null pointer or zero size");
  try {
    Limbs N(n, n + words);
    const size_t b = H::bits(N);
    if (b < 2 || !(N[0] & 1)) return fail(FLB_EINVAL, "modulus must be odd and >= 3");
    uint32_t S = 0;
    for (uint32_t f : {32u, 64u, 96u, 128u, 192u, 256u})
      if (b <= 32u * f) { S = f; break; }
    if (!S) return fail(FLB_EUNSUPPORTED, "modulus above 8192 bits");
    *out = make_mod(N, S);
    return FLB_OK;
  } catch (const std::bad_alloc&) {
    return fail(FLB_ENOMEM, "host allocation failed");
  } catch (const std::exception& ex) {
    return fail(FLB_EINVAL, ex.what());
  }
}

void flb_mod_free(flb_mod* M) { delete M; }
uint32_t flb_mod_words(const flb_mod* M) { return M ? M->core.s : 0; }

int flb_mod_mul(const flb_mod* M, const uint32_t* a, const uint32_t* b, uint32_t* out, size_t count, void* stream) {
  if (!M) return fail(FLB_EINVAL, "null modulus");
  return flb_add(&M->core, a, b, out, count, stream);
}

int flb_mod_pow(const flb_mod* M, const uint32_t* base, const uint32_t* e, uint32_t e_words, uint32_t* out,
                size_t count, void* stream) {
  if (!M) return fail(FLB_EINVAL, "null modulus");
  return flb_scalar_mul(&M->core, base, e, e_words, out, count, stream);
}

int flb_mod_pow_shared(const flb_mod* Mc, const uint32_t* base, const uint32_t* e_host, uint32_t e_words,
                       uint32_t* out, size_t count, void* stream) {
  if (!Mc || !base || !e_host || !out || e_words == 0) return fail(FLB_EINVAL, "null pointer or zero size");
  if (count == 0) return FLB_OK;
  flb_mod* M = const_cast<flb_mod*>(Mc);
  const flb_pub* K = &M->core;
  std::vector<uint32_t> e(e_host, e_host + e_words);
  while (e.size() > 1 && e.back() == 0) e.pop_back();
  if (e.size() == 1 && e[0] == 0) {  // x^0 = 1
    flb::k_fill_one<<<grid_1d(count * K->s), 256, 0, (cudaStream_t)stream>>>(out, count, K->s);
    FLB_LAUNCH_CHECK();
    return FLB_OK;
  }
  uint32_t* dev;
  int rc = const_cast<DevBlob&>(K->dev).get(K->blob, &dev);
  if (rc) return rc;
  const H::Schedule* S;
  const uint32_t* sched_dev;
  {
    std::lock_guard<std::mutex> lk(M->mu);
    auto it = M->scheds.find(e);
    if (it == M->scheds.end()) {
      try {
        it = M->scheds.emplace(e, flb_mod::Sched{H::best_schedule(Limbs(e.begin(), e.end()), 7), {}}).first;
      } catch (const std::exception& ex) {
        return fail(FLB_EINVAL, ex.what());
      }
    }
    int d;
    FLB_CK(cudaGetDevice(&d));
    auto& dv = it->second.dev;
    if (!dv.count(d)) {
      uint32_t* p = nullptr;
      const auto& ops = it->second.s.ops;
      FLB_CK(cudaMalloc(&p, ops.size() * 4));
      FLB_CK(cudaMemcpy(p, ops.data(), ops.size() * 4, cudaMemcpyHostToDevice));
      dv[d] = p;
    }
    S = &it->second.s;
    sched_dev = dv[d];
  }
  FLB_DISPATCH_ENC(K->frame, run_modpow, K, dev, sched_dev, S, base, out, count, (cudaStream_t)stream);
}

int flb_rsa_keygen(uint32_t key_bits, uint64_t seed, uint32_t e, uint32_t* n_out, uint32_t* d_out, uint32_t* p_out,
                   uint32_t* q_out) {
  if (key_bits < 64 || key_bits > 8192 || key_bits % 64 || e < 3 || !(e & 1))
    return fail(FLB_EINVAL, "key_bits must be a multiple of 64 in [64, 8192]; e odd >= 3");
  try {
    H::Xoshiro256 rng(seed ^ 0x5253412d6b657973ull);
    const uint32_t w = key_bits / 32;
    for (;;) {
      Limbs p = H::random_prime(key_bits / 2, rng), q = H::random_prime(key_bits / 2, rng);
      if (H::cmp(p, q) == 0) continue;
      if (H::cmp(p, q) < 0) std::swap(p, q);
      Limbs n = H::resized(H::mul(p, q), w);
      if (H::bits(n) != key_bits) continue;
      Limbs one(p.size(), 0);
      one[0] = 1;
      Limbs pm1 = p, qm1 = q;
      H::sub_in(pm1, one);
      H::sub_in(qm1, one);
      const Limbs phi = H::mul(pm1, qm1);
      const uint32_t r = H::mod_small(phi, e);
      if (r == 0) continue;  // gcd(e, phi) != 1 (e prime or not: require phi mod e != 0 and check below)
      // k = -phi^-1 mod e (small), d = (1 + k phi) / e
      uint64_t inv = 0;
      for (uint64_t t = 1; t < e; t++)
        if ((r * t) % e == 1) { inv = t; break; }
      if (!inv) continue;  // e not coprime to phi
      const uint32_t k = (uint32_t)((e - inv) % e);
      Limbs dnum = H::mul_small(phi, k, 1);
      if (H::mod_small(dnum, e) != 0) continue;
      Limbs d = H::resized(H::div_small(dnum, e), w + 1);
      d = H::resized(d, w);
      if (n_out) for (uint32_t i = 0; i < w; i++) n_out[i] = n[i];
      if (d_out) for (uint32_t i = 0; i < w; i++) d_out[i] = d[i];
      Limbs ph = H::resized(p, w / 2), qh = H::resized(q, w / 2);
      if (p_out) for (uint32_t i = 0; i < w / 2; i++) p_out[i] = ph[i];
      if (q_out) for (uint32_t i = 0; i < w / 2; i++) q_out[i] = qh[i];
      return FLB_OK;
    }
  } catch (const std::exception& ex) {
    return fail(FLB_EINVAL, ex.what());
  }
}

// Segmented multi-exponentiation (Hetero-LR's per-feature sum of residual x feature, C3):
// Pippenger's bucket method on top of the segmented product kernel.
int flb_multiexp_segments(const flb_pub* K, const uint32_t* c, size_t num_inputs, const int64_t* idx, const uint32_t* e,
                          uint32_t e_words, const int64_t* offsets, size_t num_segments, size_t num_entries, uint32_t* out,
                          void* stream) {
  if (!K || !offsets || !out || (num_entries && (!c || !e))) return fail(FLB_EINVAL, "null pointer");
  if (e_words < 1 || e_words > 8) return fail(FLB_EINVAL, "e_words must be in [1, 8]");
  if (num_segments == 0) return FLB_OK;
  cudaStream_t st = (cudaStream_t)stream;
  if (debug_checks()) {
    uint32_t* dev;
    int rc;
    if ((rc = pub_dev(K, &dev)) || (rc = check_segments(idx, num_entries, num_inputs, offsets, num_segments, stream)) ||
        (num_inputs && (rc = check_below(c, num_inputs, K->s, dev + K->o_n2, stream, "ciphertexts c >= n^2"))))
      return rc;
  }
  const uint32_t s_words = K->s;
  const uint64_t Kb = 32ull * e_words;
  const uint64_t avg = num_entries / num_segments;
  const char* force = getenv("FLB_MULTIEXP");
  const bool naive = (force && std::string(force) == "naive") || avg < 256;
  if (naive) {
    // gather c[idx[t]] for every entry, scalar-mul by e_t, product per segment
    Scratch rows, pw;
    int rc = rows.alloc(std::max<size_t>(1, num_entries) * s_words * 4, st);
    if (rc) return rc;
    rc = pw.alloc(std::max<size_t>(1, num_entries) * s_words * 4, st);
    if (rc) return rc;
    if (num_entries) {
      flb::k_gather_rows<<<grid_1d(num_entries * s_words), 256, 0, st>>>(c, idx, (int64_t)num_entries, s_words,
                                                                          (uint32_t*)rows.p);
      FLB_LAUNCH_CHECK();
      rc = flb_scalar_mul(K, (const uint32_t*)rows.p, e, e_words, (uint32_t*)pw.p, num_entries, stream);
      if (rc) return rc;
    }
    return flb_reduce_segments(K, (const uint32_t*)pw.p, num_entries, nullptr, num_entries, offsets, num_segments, 0,
                               out, stream);
  }
  // window width minimising entries*W (bucket products) + W*cb*2^(cb-1) (bit planes), bucket count capped
  uint32_t cb = 4;
  double best = 1e300;
  for (uint32_t t = 4; t <= 16; t++) {
    const uint64_t W = (Kb + t - 1) / t;
    if ((uint64_t)num_segments * W << t > (8ull << 20)) break;
    const double cost = (double)num_entries * W + (double)num_segments * W * t * (double)(1ull << (t - 1));
    if (cost < best) { best = cost; cb = t; }
  }
  const uint64_t W = (Kb + cb - 1) / cb;
  const uint64_t nb = (uint64_t)num_segments * W << cb;
  const uint64_t planes = W * cb, nplanes = (uint64_t)num_segments * planes, half = 1ull << (cb - 1);
  Scratch s_cnt, s_off, s_sorted, s_B, s_idx2, s_off2, s_P;
  int rc;
  if ((rc = s_cnt.alloc((nb + 1) * 8, st)) || (rc = s_off.alloc((nb + 1) * 8, st)) ||
      (rc = s_sorted.alloc(std::max<uint64_t>(1, num_entries * W) * 8, st)) || (rc = s_B.alloc(nb * s_words * 4, st)) ||
      (rc = s_idx2.alloc(nplanes * half * 8, st)) || (rc = s_off2.alloc((nplanes + 1) * 8, st)) ||
      (rc = s_P.alloc(nplanes * s_words * 4, st)))
    return rc;
  unsigned long long* cnt = (unsigned long long*)s_cnt.p;
  int64_t* boff = (int64_t*)s_off.p;
  FLB_CK(cudaMemsetAsync(cnt, 0, (nb + 1) * 8, st));
  const int g = grid_1d(num_entries);
  if (num_entries) {
    flb::k_bucket<0><<<g, 256, 0, st>>>(offsets, (int64_t)num_segments, (int64_t)num_entries, idx, e, e_words,
                                        (uint32_t)W, cb, cnt, nullptr);
    FLB_LAUNCH_CHECK();
  }
  flb::k_scan_u64<<<1, 1024, 0, st>>>(cnt, (int64_t)nb, boff);
  FLB_LAUNCH_CHECK();
  FLB_CK(cudaMemcpyAsync(cnt, boff, nb * 8, cudaMemcpyDeviceToDevice, st));  // cursors = bucket starts
  if (num_entries) {
    flb::k_bucket<1><<<g, 256, 0, st>>>(offsets, (int64_t)num_segments, (int64_t)num_entries, idx, e, e_words,
                                        (uint32_t)W, cb, cnt, (int64_t*)s_sorted.p);
    FLB_LAUNCH_CHECK();
  }
  // bucket products, then bit-plane products, then Horner over the planes
  rc = flb_reduce_segments(K, c, num_inputs, (const int64_t*)s_sorted.p, std::max<uint64_t>(1, num_entries * W), boff,
                           nb, 0, (uint32_t*)s_B.p, stream);
  if (rc) return rc;
  flb::k_bitplane_index<<<grid_1d(nplanes * half), 256, 0, st>>>((int64_t)nplanes, cb, (int64_t*)s_idx2.p);
  FLB_LAUNCH_CHECK();
  flb::k_arange_offsets<<<grid_1d(nplanes + 1), 256, 0, st>>>((int64_t)nplanes, (int64_t)half, (int64_t*)s_off2.p);
  FLB_LAUNCH_CHECK();
  rc = flb_reduce_segments(K, (const uint32_t*)s_B.p, nb, (const int64_t*)s_idx2.p, nplanes * half,
                           (const int64_t*)s_off2.p, nplanes, half, (uint32_t*)s_P.p, stream);
  if (rc) return rc;
  uint32_t* dev;
  rc = const_cast<DevBlob&>(K->dev).get(K->blob, &dev);
  if (rc) return rc;
  FLB_DISPATCH_ENC(K->frame, run_horner, K, dev, (const uint32_t*)s_P.p, (uint32_t)planes, out, num_segments, st);
}

static int frame_key(uint32_t words, uint32_t* key);

static int crt_pre_dispatch(const flb_priv* V, const uint32_t* dev, const uint32_t* r, uint64_t seed, uint64_t ctr0,
                            uint32_t* y, size_t count, cudaStream_t st) {
  uint32_t key;
  int rc = frame_key(V->H, &key);
  if (rc) return rc;
  FLB_DISPATCH_ENC(key, run_crt_pre, V, dev, r, seed, ctr0, y, count, st);
}

static int crt2_dispatch(const flb_priv* V, const uint32_t* dev, const uint32_t* m, const uint32_t* y, uint32_t* c,
                         size_t count, cudaStream_t st) {
  FLB_DISPATCH_DEC(V->pub->frame, run_encrypt_crt2, V, dev, m, y, c, count, st);
}

static int encrypt_crt_v2(const flb_priv* V, const uint32_t* dev, const uint32_t* m, const uint32_t* r, uint64_t seed,
                          uint64_t ctr0, uint32_t* c, size_t count, cudaStream_t st) {
  if (use_tc(V) && use_tc_half(V) && V->H == 32 && V->pub->sp == 64 && tc_dag_enabled())
    return run_encrypt_kh_dag<32, 64>(V, dev, m, r, seed, ctr0, c, count, st);  // 2048-bit keys: one launch
  Scratch ys;
  int rc = ys.alloc((size_t)2 * count * V->H * 4, st);
  if (rc) return rc;
  if (use_tc_half(V))
    rc = V->H == 64 ? run_crt_pre_tc<64>(V, dev, r, seed, ctr0, (uint32_t*)ys.p, count, st)
                    : run_crt_pre_tc<32>(V, dev, r, seed, ctr0, (uint32_t*)ys.p, count, st);
  else
    rc = crt_pre_dispatch(V, dev, r, seed, ctr0, (uint32_t*)ys.p, count, st);
  if (rc) return rc;
  if (use_tc(V)) {
    if (V->pub->sp == 128) return run_encrypt_crt_tc<128>(V, dev, m, (const uint32_t*)ys.p, c, count, st);
    if (V->pub->sp == 96) return run_encrypt_crt_tc<96>(V, dev, m, (const uint32_t*)ys.p, c, count, st);
    if (V->pub->sp == 64) return run_encrypt_crt_tc<64>(V, dev, m, (const uint32_t*)ys.p, c, count, st);
    return run_encrypt_crt_tc<32>(V, dev, m, (const uint32_t*)ys.p, c, count, st);
  }
  return crt2_dispatch(V, dev, m, (const uint32_t*)ys.p, c, count, st);
}

static int frame_key(uint32_t words, uint32_t* key) {
  switch (words) {
    case 32: *key = 512; return FLB_OK;
    case 64: *key = 1024; return FLB_OK;
    case 96: *key = 1536; return FLB_OK;
    case 128: *key = 2048; return FLB_OK;
    case 192: *key = 3072; return FLB_OK;
    case 256: *key = 4096; return FLB_OK;
  }
  return fail(FLB_EINVAL, "words must be one of 32, 64, 96, 128, 192, 256");
}

int flb_miller_rabin(const uint32_t* cand, uint32_t words, const uint32_t* mont_bases, uint32_t rounds, uint64_t seed,
                     uint32_t* verdict, size_t count, void* stream) {
  if (!cand || !verdict || rounds == 0 || rounds > 64) return fail(FLB_EINVAL, "null pointer or rounds not in [1, 64]");
  uint32_t key;
  int rc = frame_key(words, &key);
  if (rc) return rc;
  if (count == 0) return FLB_OK;
  const int bw = 5;
  FLB_DISPATCH_ENC(key, run_mr, cand, mont_bases, rounds, seed, 0, verdict, count, bw, (cudaStream_t)stream);
}

int flb_keygen_gpu(uint32_t key_bits, uint64_t seed, flb_pub** pub, flb_priv** priv, void* stream) {
  if (!pub || !priv) return fail(FLB_EINVAL, "null output pointer");
  if (key_bits != 1024 && key_bits != 2048 && key_bits != 3072 && key_bits != 4096)
    return fail(FLB_EINVAL, "key_bits must be 1024, 2048, 3072 or 4096");
  cudaStream_t st = (cudaStream_t)stream;
  const uint32_t pbits = key_bits / 2, pwords = (pbits + 31) / 32;
  uint32_t S = 32;
  while (S < pwords) S += 32;
  if (S == 160 || S == 224) S += 32;
  uint32_t key;
  int rc = frame_key(S, &key);
  if (rc) return rc;
  const uint64_t B = 8192;  // candidates per batch
  std::vector<uint32_t> primes;
  for (uint32_t p : H::small_primes()) primes.push_back(p);
  uint32_t *d_cand = nullptr, *d_flag = nullptr, *d_primes = nullptr, *d_surv = nullptr, *d_ver = nullptr;
  auto cleanup = [&] {
    cudaFree(d_cand); cudaFree(d_flag); cudaFree(d_primes); cudaFree(d_surv); cudaFree(d_ver);
  };
  auto ck = [&](cudaError_t e, const char* what) {
    if (e != cudaSuccess) {
      g_err = std::string(what) + ": " + cudaGetErrorString(e);
      cleanup();
      return FLB_ECUDA;
    }
    return FLB_OK;
  };
  if ((rc = ck(cudaMalloc(&d_cand, B * S * 4), "cudaMalloc")) || (rc = ck(cudaMalloc(&d_flag, B * 4), "cudaMalloc")) ||
      (rc = ck(cudaMalloc(&d_primes, primes.size() * 4), "cudaMalloc")) ||
      (rc = ck(cudaMalloc(&d_surv, B * S * 4), "cudaMalloc")) || (rc = ck(cudaMalloc(&d_ver, B * 4), "cudaMalloc")))
    return rc;
  if ((rc = ck(cudaMemcpy(d_primes, primes.data(), primes.size() * 4, cudaMemcpyHostToDevice), "cudaMemcpy"))) return rc;
  std::vector<uint32_t> flags(B), ver(B), host_c(B * S);
  std::vector<Limbs> found;
  for (uint64_t batch = 0; found.size() < 2 && batch < 4096; batch++) {
    flb::k_gen_candidates<<<grid_1d(B * S), 256, 0, st>>>(d_cand, B, S, pbits, seed, batch * B);
    flb::k_sieve<<<grid_1d(B), 256, 0, st>>>(d_cand, B, S, pwords, d_primes, (uint32_t)primes.size(), d_flag);
    if ((rc = ck(cudaGetLastError(), "launch")) || (rc = ck(cudaMemcpyAsync(flags.data(), d_flag, B * 4,
                                                                            cudaMemcpyDeviceToHost, st), "copy")) ||
        (rc = ck(cudaMemcpyAsync(host_c.data(), d_cand, B * S * 4, cudaMemcpyDeviceToHost, st), "copy")) ||
        (rc = ck(cudaStreamSynchronize(st), "sync")))
      return rc;
    std::vector<uint64_t> idx;
    for (uint64_t i = 0; i < B; i++)
      if (flags[i]) idx.push_back(i);
    // round 1 on every sieve survivor, then 39 more on the passers (Miller–Rabin)
    for (int phase = 0; phase < 2 && !idx.empty(); phase++) {
      std::vector<uint32_t> surv(idx.size() * S);
      for (size_t t = 0; t < idx.size(); t++)
        std::memcpy(&surv[t * S], &host_c[idx[t] * S], S * 4);
      if ((rc = ck(cudaMemcpyAsync(d_surv, surv.data(), surv.size() * 4, cudaMemcpyHostToDevice, st), "copy"))) return rc;
      const uint32_t rounds = phase == 0 ? 1 : 39;
      rc = flb_miller_rabin(d_surv, S, nullptr, rounds, seed ^ (0x4d52000000000000ull + batch * 2 + phase), d_ver,
                            idx.size(), stream);
      if (rc) { cleanup(); return rc; }
      if ((rc = ck(cudaMemcpyAsync(ver.data(), d_ver, idx.size() * 4, cudaMemcpyDeviceToHost, st), "copy")) ||
          (rc = ck(cudaStreamSynchronize(st), "sync")))
        return rc;
      std::vector<uint64_t> keep;
      for (size_t t = 0; t < idx.size(); t++)
        if (ver[t]) keep.push_back(idx[t]);
      idx.swap(keep);
    }
    for (uint64_t i : idx) {
      Limbs p(host_c.begin() + i * S, host_c.begin() + i * S + pwords);
      if (found.empty() || H::cmp(found[0], p) != 0) found.push_back(p);
      if (found.size() == 2) break;
    }
  }
  cleanup();
  if (found.size() < 2) return fail(FLB_EKEY, "no primes found");
  try {
    flb_priv* V = make_priv(found[0], found[1]);
    *priv = V;
    *pub = make_pub(V->pub->n);
  } catch (const std::exception& ex) {
    return fail(FLB_EKEY, ex.what());
  }
  return FLB_OK;
}

static int codec_args(const flb_pub* K, const flb_codec* cd, flb::CodecArgs* A) {
  if (!cd) return fail(FLB_EINVAL, "null codec");
  if (cd->qbits < 1 || cd->qbits > 52) return fail(FLB_EINVAL, "qbits must be in [1, 52]");
  if (cd->slot_bits != cd->qbits + cd->pad_bits) return fail(FLB_EINVAL, "slot_bits != qbits + pad_bits");
  if (cd->slot_bits != 32 && cd->slot_bits != 64) return fail(FLB_EINVAL, "slot_bits must be 32 or 64");
  if (cd->slots < 1 || cd->slots > flb_slot_capacity(K, cd->slot_bits))
    return fail(FLB_EINVAL, "slots must be in [1, floor((bits(n)-1)/slot_bits)]");
  if (!(cd->alpha > 0.0)) return fail(FLB_EINVAL, "alpha must be > 0");
  A->alpha = cd->alpha;
  A->sigma = (double)((1ull << cd->qbits) - 1) / (2.0 * cd->alpha);
  A->qbits = cd->qbits;
  A->slot_words = cd->slot_bits / 32;
  A->slots = cd->slots;
  A->pt_words = K->sp;
  A->qmax = (1ull << cd->qbits) - 1;
  return FLB_OK;
}

static int grid_1d(uint64_t n) {
  int dev, sms = 148;
  if (cudaGetDevice(&dev) == cudaSuccess) cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  const uint64_t want = (n + 255) / 256;
  return (int)std::max<uint64_t>(1, std::min<uint64_t>(want, (uint64_t)sms * 8));
}

int flb_pack(const flb_pub* K, const flb_codec* cd, const float* x, size_t n_values, uint32_t* pt, void* stream) {
  if (!K || !x || !pt) return fail(FLB_EINVAL, "null pointer");
  flb::CodecArgs A;
  int rc = codec_args(K, cd, &A);
  if (rc) return rc;
  if (n_values == 0) return FLB_OK;
  const uint64_t n_pt = (n_values + A.slots - 1) / A.slots;
  flb::k_pack<<<grid_1d(n_pt * A.pt_words), 256, 0, (cudaStream_t)stream>>>(x, n_values, n_pt, A, pt);
  FLB_LAUNCH_CHECK();
  return FLB_OK;
}

int flb_unpack(const flb_pub* K, const flb_codec* cd, const uint32_t* pt, size_t n_values, const uint32_t* summands,
               uint32_t summands_scalar, float* x, void* stream) {
  if (!K || !x || !pt) return fail(FLB_EINVAL, "null pointer");
  flb::CodecArgs A;
  int rc = codec_args(K, cd, &A);
  if (rc) return rc;
  // the b = pad_bits overflow bits hold at most 2^b summands per slot
  const uint64_t cap = cd->pad_bits >= 63 ? ~0ull : (1ull << cd->pad_bits);
  if (!summands && (uint64_t)summands_scalar > cap) return fail(FLB_EINVAL, "summands > 2^pad_bits (slot overflow)");
  if (n_values == 0) return FLB_OK;
  if (summands && debug_checks()) {
    const uint64_t n_pt = (n_values + A.slots - 1) / A.slots;
    cudaStream_t st = (cudaStream_t)stream;
    rc = run_check(st, "summands > 2^pad_bits (slot overflow)", [&](unsigned long long* d) {
      flb::k_check_counts<<<grid_1d(n_pt), 256, 0, st>>>(summands, n_pt, cap, d);
    });
    if (rc) return rc;
  }
  flb::k_unpack<<<grid_1d(n_values), 256, 0, (cudaStream_t)stream>>>(pt, n_values, A, summands, summands_scalar, x);
  FLB_LAUNCH_CHECK();
  return FLB_OK;
}

int flb_unpack_sums(const flb_pub* K, const flb_codec* cd, const uint32_t* pt, size_t n_values, uint64_t* sums,
                    void* stream) {
  if (!K || !sums || !pt) return fail(FLB_EINVAL, "null pointer");
  flb::CodecArgs A;
  int rc = codec_args(K, cd, &A);
  if (rc) return rc;
  if (n_values == 0) return FLB_OK;
  flb::k_unpack_sums<<<grid_1d(n_values), 256, 0, (cudaStream_t)stream>>>(pt, n_values, A,
                                                                          (unsigned long long*)sums);
  FLB_LAUNCH_CHECK();
  return FLB_OK;
}

}  // extern "C"
