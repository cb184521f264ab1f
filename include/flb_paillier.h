/* flb_paillier.h — C ABI of the B200 batched-Paillier library (FLBooster hot path).
 *
 * Paper: Zeng et al., "FLBooster: A Unified and Efficient Platform for Federated Learning
 * Acceleration", ICDE 2023 — cited as PAPER L<line> of /root/reference/PAPER.md.
 * This header is the boundary of SURVEY.md §8(b): Table I's Paillier rows (PAPER L252–L256:
 * key_gen, encrypt, decrypt, add) batched over device pointers, plus scalar_mul, pack/unpack
 * (PAPER §IV-B/§IV-C, Eq. 6–9) and a segmented ciphertext-product reduction.
 *
 * Conventions shared by every entry point
 * ---------------------------------------
 *  - Big integers are little-endian 32-bit limbs (base 2^w, w = 32), stored
 *    row-major [count][words].  Plaintexts use pt_words = k/32 limbs and ciphertexts
 *    ct_words = k/16 limbs, where k is the key's frame (1024, 2048, 3072 or 4096; smaller
 *    "toy" keys are padded into the 1024 frame).  Buffers must be 16-byte aligned.
 *  - Batch pointers are DEVICE pointers owned by the caller; every batch call is enqueued on
 *    `stream` (a cudaStream_t passed as void*; NULL = legacy default stream) and returns
 *    without synchronising.  The device is the caller's current CUDA device.  Scratch (window
 *    tables, reduction partials) is taken from the device's stream-ordered pool on `stream`
 *    and returned on the same stream.  Device faults surface at stream synchronisation.
 *  - Key handles are immutable after creation and thread-safe; their constants are uploaded
 *    to a device on first use there (a one-time synchronous copy).
 *  - Status: FLB_OK (0) or a negative FLB_E* code; flb_last_error() gives a thread-local
 *    message for the last failure.  Argument errors are detected before any launch.  Value
 *    ranges (m < n, c < n^2, gcd(r, n) = 1) are NOT checked on the hot path: encrypt, add,
 *    scalar_mul and reduce return the mathematical function of the given integers; decrypt is
 *    specified for units c of Z_{n^2} (every unit is a valid ciphertext) and its
 *    output for a non-unit is unspecified.
 *  - FLB_DEBUG_CHECKS=1 in the environment (read per call) turns on device-side range checks
 *    before the op: plaintexts m < n (encrypt, encrypt_crt), ciphertexts c < n^2 (decrypt, add,
 *    scalar_mul, reduce_segments, multiexp_segments; the modulus for flb_mod_*), offsets well
 *    formed and idx in [0, num_inputs) (reduce_segments, multiexp_segments), per-plaintext
 *    summands <= 2^pad_bits (unpack).  The call then synchronises `stream` and returns
 *    FLB_EINVAL naming the violation and the number of offending elements.  gcd(r, n) = 1 is
 *    not checked (probability of a violation ~2^(1-k/2), reading c4).
 */
#ifndef FLB_PAILLIER_H
#define FLB_PAILLIER_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct flb_pub flb_pub;   /* n, n^2, Montgomery constants, encryption schedule */
typedef struct flb_priv flb_priv; /* p, q, p^2, q^2, CRT constants, decryption schedules */
typedef struct flb_mod flb_mod;   /* any odd modulus (Table I mod_mul / mod_pow, RSA)             */

enum {
  FLB_OK = 0,
  FLB_EINVAL = -1,      /* bad argument (null pointer, unsupported size, bad codec) */
  FLB_ENOMEM = -2,      /* host or device allocation failed */
  FLB_ECUDA = -3,       /* a CUDA call or kernel launch failed */
  FLB_EKEY = -4,        /* key material rejected (not prime, p == q, gcd(n, phi) != 1) */
  FLB_EUNSUPPORTED = -5 /* modulus larger than 4096 bits */
};

/* ---------------------------------------------------------------- keys (host, not timed) */

/* Paillier::key_gen(size) (key generation L89).  Deterministic in `seed`:
 * xoshiro256** candidates with the top two bits and the low bit set, small-prime sieve,
 * 40-round Miller–Rabin.  key_bits in {1024, 2048, 3072, 4096}; p, q have
 * key_bits/2 bits, bits(n) = key_bits, g = n + 1.  On success *pub and *priv are new handles
 * (free with flb_pub_free / flb_priv_free).  Errors: FLB_EINVAL. */
int flb_keygen(uint32_t key_bits, uint64_t seed, flb_pub** pub, flb_priv** priv);

/* Import a key from its primes (host little-endian limbs, prime_words each).  The larger prime
 * becomes p.  bits(n) <= 4096; keys below 1024 bits use the 1024 frame.  Errors: FLB_EINVAL
 * (null / zero size), FLB_EKEY (p == q, a prime even or < 3, a prime failing Miller–Rabin,
 * gcd(n, (p-1)(q-1)) != 1), FLB_EUNSUPPORTED (bits(n) > 4096). */
int flb_key_from_primes(const uint32_t* p, const uint32_t* q, uint32_t prime_words,
                        flb_pub** pub, flb_priv** priv);

/* Copy p, q (prime_words(pub)= pt_words/2 limbs each) and n (pt_words limbs) to host
 * buffers; any output pointer may be NULL. */
int flb_key_export(const flb_priv* priv, uint32_t* p, uint32_t* q, uint32_t* n);

void flb_pub_free(flb_pub* pub);
void flb_priv_free(flb_priv* priv);

uint32_t flb_key_bits(const flb_pub* pub);  /* bits(n) */
uint32_t flb_pt_words(const flb_pub* pub);  /* frame/32 */
uint32_t flb_ct_words(const flb_pub* pub);  /* frame/16 */
/* floor((bits(n) - 1) / slot_bits): slots per plaintext that cannot wrap mod n (reading c16 of
 * PAPER L258). */
uint32_t flb_slot_capacity(const flb_pub* pub, uint32_t slot_bits);

/* ---------------------------------------------------------------- batched device ops */

/* Paillier::encrypt (Eq. 3): c_i = g^{m_i} r_i^n mod n^2 with g = n+1,
 * computed as (1 + m_i n) r_i^n.  m: [count][pt_words], each m_i < n.  r: [count][pt_words]
 * caller randomness (each r_i < n, gcd(r_i, n) = 1), or NULL to draw r_i on the device from
 * Philox4x32-10 with key = seed and counter (ctr0 + i, j) exactly as oracle/philox.py draw_r
 * (reading c4).  c: [count][ct_words].  count = 0 is a no-op.  For 1024/2048-bit keys (n^2 of 64/128
 * words) a batch of at least 96 elements per SM runs on the tensor-core Montgomery kernel (see
 * flb_encrypt_crt); smaller batches, FLB_TC=0 and larger keys run the CIOS kernel (same bits;
 * FLB_TC=2 forces the tensor cores at any size).  Errors: FLB_EINVAL, FLB_ECUDA. */
int flb_encrypt(const flb_pub* pub, const uint32_t* m, const uint32_t* r, uint64_t seed,
                uint64_t ctr0, uint32_t* c, size_t count, void* stream);

/* Encryption by a holder of the private key: the same c_i as flb_encrypt (same m, r, seed,
 * ctr0 -> the same bits), computed as (1 + m n) r^n mod p^2 and mod q^2 with half-size moduli and
 * recombined by CRT (c = c_q + q^2 ((c_p - c_q) (q^2)^-1 mod p^2)) — about half the limb products.
 * Beyond the paper; in Fig. 2 the clients that encrypt also
 * decrypt, so they hold the key.  From 2048 bits the exponentiation is two-stage,
 * r^n mod P^2 = (r^Q mod P)^P mod P^2; for 1024-4096-bit keys (P^2 of 32/64/96/128 words) and the
 * half-frame first stage at 2048-4096 bits every Montgomery product runs its reduction
 * q = t N' mod R, (t + q N)/R as u8 tcgen05 MMAs against Toeplitz matrices of N' and N (the batch
 * shares N) with TMEM accumulators (csrc/flb_tc.cuh); FLB_TC=0 in the environment selects the
 * CUDA-core CIOS kernels (same bits).  Scratch: stream-ordered, about 2 count (ct_words) words.
 * Arguments and errors as flb_encrypt. */
int flb_encrypt_crt(const flb_priv* priv, const uint32_t* m, const uint32_t* r, uint64_t seed,
                    uint64_t ctr0, uint32_t* c, size_t count, void* stream);

/* Paillier::decrypt (Eq. 4), by CRT (reading c10).  c: [count][ct_words]
 * (each a unit < n^2), m: [count][pt_words] receives m_i in [0, n).  For 1024/2048-bit keys the two
 * exponentiations c^(P-1) mod P^2 run on the tensor-core Montgomery kernel (3072/4096-bit keys too:
 * P^2 of 96/128 words; see flb_encrypt_crt; FLB_TC=0 selects CIOS, same bits).  Errors: FLB_EINVAL, FLB_ECUDA. */
int flb_decrypt(const flb_priv* priv, const uint32_t* c, uint32_t* m, size_t count, void* stream);

/* Paillier::add (Eq. 5): out_i = c1_i * c2_i mod n^2.  All
 * [count][ct_words]; out may alias c1 or c2.  Errors: FLB_EINVAL, FLB_ECUDA. */
int flb_add(const flb_pub* pub, const uint32_t* c1, const uint32_t* c2, uint32_t* out,
            size_t count, void* stream);

/* Homomorphic scalar multiply (mod_pow; reading c19): out_i = c_i^{e_i} mod n^2
 * = E(e_i m_i).  e: [count][e_words] unsigned little-endian exponents (1 <= e_words <= 128);
 * e_i = 0 gives 1.  c, out: [count][ct_words] (no aliasing).  Errors: FLB_EINVAL, FLB_ECUDA. */
int flb_scalar_mul(const flb_pub* pub, const uint32_t* c, const uint32_t* e, uint32_t e_words,
                   uint32_t* out, size_t count, void* stream);

/* Segmented ciphertext product (Fig. 2 server aggregation; repeated Eq. 5):
 * out_j = prod_{t = offsets[j]}^{offsets[j+1]-1} c[idx ? idx[t] : t] mod n^2, out_j = 1 for an
 * empty segment.  c: [num_inputs][ct_words]; idx: device int64 [num_entries] (entries may repeat
 * inputs) or NULL (then entry t is input t and num_entries <= num_inputs); offsets: device int64
 * [num_segments+1], non-decreasing, offsets[0] = 0, offsets[num_segments] = num_entries (host
 * value passed in num_entries, it sizes the scratch).  max_segment_len: an upper bound on any
 * segment's length if known (sizes the number of reduction levels), 0 = unknown (num_entries).
 * out: [num_segments][ct_words], must not alias c.  Errors: FLB_EINVAL, FLB_ECUDA. */
int flb_reduce_segments(const flb_pub* pub, const uint32_t* c, size_t num_inputs,
                        const int64_t* idx, size_t num_entries, const int64_t* offsets,
                        size_t num_segments, size_t max_segment_len, uint32_t* out, void* stream);

/* Segmented multi-exponentiation: out_j = prod_{t = offsets[j]}^{offsets[j+1]-1} c[idx ? idx[t] : t]^(e_t)
 * mod n^2 = E(sum_t e_t m_t) — Hetero-LR's per-feature sum of encrypted residuals x feature values
 * (PAPER L375 models; Table I mod_pow, L246, composed with Eq. 5).  e: device [num_entries][e_words]
 * (1 <= e_words <= 8), one exponent per entry; num_entries = offsets[num_segments].  Long segments
 * use Pippenger's bucket method (digit buckets and bit-plane products are segmented products);
 * short ones scalar-mul + product.  Results are identical either way.  Scratch ~ (num_entries * W * 8
 * + buckets * ct_words * 4) bytes from the stream-ordered pool.  Errors: FLB_EINVAL, FLB_ECUDA. */
int flb_multiexp_segments(const flb_pub* pub, const uint32_t* c, size_t num_inputs, const int64_t* idx,
                          const uint32_t* e, uint32_t e_words, const int64_t* offsets,
                          size_t num_segments, size_t num_entries, uint32_t* out, void* stream);

/* Encoding-quantisation + batch compression parameters (PAPER §IV-B/§IV-C):
 * alpha: gradient bound (Eq. 6), qbits: r of Eq. 7 (L221, 1..52), pad_bits: b of Eq. 8
 * (L223), slot_bits = qbits + pad_bits in {32, 64} (L331: "a multiple of 32"), slots: values
 * per plaintext (1 <= slots <= flb_slot_capacity). */
typedef struct {
  double alpha;
  uint32_t qbits, pad_bits, slot_bits, slots;
} flb_codec;

/* Quantise + pack (Eq. 6–9; readings c11, c13, c17): x: device float32 [n_values];
 * pt: [ceil(n_values/slots)][pt_words]; plaintext j = sum_i q_{j*slots+i} 2^((slots-1-i) w).
 * Errors: FLB_EINVAL, FLB_ECUDA. */
int flb_pack(const flb_pub* pub, const flb_codec* codec, const float* x, size_t n_values,
             uint32_t* pt, void* stream);

/* Unpack + dequantise (reading c14): x_i = Sum_i / sigma - cnt * alpha in binary64,
 * rounded to float32, with cnt = summands[i / slots] (device uint32 [num_pt]) or
 * summands_scalar when summands is NULL.  cnt <= 2^pad_bits: the b = pad_bits overflow bits of a
 * slot hold at most 2^b summands "so that no overflow or inconsistent decryption results occur"
 * (reading c15).  Errors: FLB_EINVAL (also summands_scalar > 2^pad_bits; a device
 * array is checked only under FLB_DEBUG_CHECKS), FLB_ECUDA. */
int flb_unpack(const flb_pub* pub, const flb_codec* codec, const uint32_t* pt, size_t n_values,
               const uint32_t* summands, uint32_t summands_scalar, float* x, void* stream);

/* The exact slot integers Sum_i (device uint64 [n_values]).  Errors: FLB_EINVAL, FLB_ECUDA. */
int flb_unpack_sums(const flb_pub* pub, const flb_codec* codec, const uint32_t* pt,
                    size_t n_values, uint64_t* sums, void* stream);

/* ---------------------------------------------------------------- generic modular API, RSA (NEXT-4)
 * PAPER Table I (L236–L256) and §IV-D (L269–L284): mod_mul(values1, values2, n) and
 * mod_pow(x, p, n) over batches, with the same thread-group Montgomery kernels; RSA (L247–L251)
 * is key_gen below + mod_pow_shared (encrypt m^e, decrypt c^d) + mod_mul (the multiplicative
 * homomorphism).  A modulus of W limbs uses the smallest frame of 32/64/96/128/192/256 limbs >= W;
 * batch operands are [count][flb_mod_words] limbs, each < n. */

/* Create a modulus handle from host limbs (odd n >= 3, at most 8192 bits).  Errors: FLB_EINVAL,
 * FLB_EUNSUPPORTED (> 8192 bits). */
int flb_mod_create(const uint32_t* n, uint32_t words, flb_mod** out);
void flb_mod_free(flb_mod* mod);
uint32_t flb_mod_words(const flb_mod* mod); /* frame limbs of a batch element */

/* out_i = a_i b_i mod n (Table I mod_mul, L245; RSA::mul, L250). */
int flb_mod_mul(const flb_mod* mod, const uint32_t* a, const uint32_t* b, uint32_t* out,
                size_t count, void* stream);

/* out_i = base_i ^ e_i mod n with per-element exponents e [count][e_words] on the device
 * (Table I mod_pow, L246); e_i = 0 gives 1. */
int flb_mod_pow(const flb_mod* mod, const uint32_t* base, const uint32_t* e, uint32_t e_words,
                uint32_t* out, size_t count, void* stream);

/* out_i = base_i ^ e mod n with one exponent for the batch, given in HOST memory (its sliding-
 * window schedule is built once per exponent and cached on the handle): RSA::encrypt (e) and
 * RSA::decrypt (d), L248–L249. */
int flb_mod_pow_shared(const flb_mod* mod, const uint32_t* base, const uint32_t* e_host,
                       uint32_t e_words, uint32_t* out, size_t count, void* stream);

/* RSA::key_gen (L247, L281), host, deterministic in seed: p > q primes of key_bits/2 bits
 * (Miller–Rabin), n = p q with bits(n) = key_bits, d = e^-1 mod (p-1)(q-1).  n_out, d_out:
 * key_bits/32 limbs; p_out, q_out: key_bits/64 limbs (any may be NULL). */
int flb_rsa_keygen(uint32_t key_bits, uint64_t seed, uint32_t e, uint32_t* n_out, uint32_t* d_out,
                   uint32_t* p_out, uint32_t* q_out);

/* ---------------------------------------------------------------- Table I fundamentals (NEXT-4)
 * PAPER Table I (L241–L244) and §IV-D (L269–L273): "add/sub/mul/div ... compute the addition,
 * subtraction, multiplication, and division of two multi-precision integer arrays", "mod computes
 * the remainder", "mod_inv computes the modular inverse ... used to generate key pair[s]".
 * Element-wise over batches of UNSIGNED integers: every operand is a device array
 * [count][words] of little-endian u32 limbs, 1 <= words <= 256 (any width; rows 16-byte aligned
 * when words % 4 == 0, else read limb by limb).  Each element runs on a group of lanes in the
 * smallest frame of 32/64/128/256 limbs >= words (csrc/flb_mp.cu).  Asynchronous on `stream`.
 * Errors: FLB_EINVAL (null pointer, words outside [1, 256]), FLB_ECUDA. */

/* out_i = (a_i + b_i) mod 2^(32 words); carry (optional, uint32 [count]) = the carry out (0/1). */
int flb_mp_add(const uint32_t* a, const uint32_t* b, uint32_t* out, uint32_t* carry, uint32_t words,
               size_t count, void* stream);

/* out_i = (a_i - b_i) mod 2^(32 words); borrow (optional) = 1 iff a_i < b_i. */
int flb_mp_sub(const uint32_t* a, const uint32_t* b, uint32_t* out, uint32_t* borrow, uint32_t words,
               size_t count, void* stream);

/* out_i = a_i b_i, the full product: out is [count][2 words]. */
int flb_mp_mul(const uint32_t* a, const uint32_t* b, uint32_t* out, uint32_t words, size_t count,
               void* stream);

/* q_i = floor(a_i / b_i), r_i = a_i mod b_i (either output may be NULL, not both); b_i = 0 gives
 * q_i = 2^(32 words) - 1 and r_i = a_i (binary restoring division with a zero divisor). */
int flb_mp_divmod(const uint32_t* a, const uint32_t* b, uint32_t* q, uint32_t* r, uint32_t words,
                  size_t count, void* stream);

/* Table I mod(x, n): r_i = x_i mod n_i (flb_mp_divmod's remainder; n_i = 0 gives x_i). */
int flb_mp_mod(const uint32_t* x, const uint32_t* n, uint32_t* r, uint32_t words, size_t count,
               void* stream);

/* Table I mod_inv(x, n): out_i = x_i^-1 mod n_i in [1, n_i) when n_i >= 2 and gcd(x_i, n_i) = 1
 * (any n_i, odd or even, e.g. d = e^-1 mod phi(n) for RSA); otherwise out_i = 0.  ok (optional,
 * uint32 [count]) = 1 iff the inverse exists. */
int flb_mp_mod_inv(const uint32_t* x, const uint32_t* n, uint32_t* out, uint32_t* ok, uint32_t words,
                   size_t count, void* stream);

/* ---------------------------------------------------------------- GPU key generation (NEXT-3)
 * "random number generator for large integers (including Miller-Rabin large prime
 * number generator)".  flb_miller_rabin runs `rounds` Miller–Rabin rounds on a batch of odd
 * candidates (device [count][words], words in {32, 64, 96, 128, 192, 256}, each >= 5), each with
 * its own modulus; verdict[i] = 1 iff candidate i passed every round.  mont_bases: device
 * [count][rounds][words] bases in Montgomery form (a~ with 1 <= a~ < P stands for the base
 * a = a~ 2^(-32 words) mod P), or NULL to draw them from Philox(seed, i, round).
 * flb_keygen_gpu: Paillier::key_gen on the device — Philox candidates with the top two bits and
 * bit 0 set, a small-prime sieve kernel, one Miller–Rabin round on every survivor and 39 more on
 * the passers; the first two distinct probable primes (in candidate order) make the key, so the
 * result is deterministic in seed (a different stream of primes from flb_keygen). */
int flb_miller_rabin(const uint32_t* cand, uint32_t words, const uint32_t* mont_bases, uint32_t rounds,
                     uint64_t seed, uint32_t* verdict, size_t count, void* stream);
int flb_keygen_gpu(uint32_t key_bits, uint64_t seed, flb_pub** pub, flb_priv** priv, void* stream);

/* ---------------------------------------------------------------- host-buffer pipeline (NEXT-1)
 * PAPER Fig. 4 / §V-A (L288–L298): host data -> compression -> copy to GPU -> HE -> copy back.
 * These take HOST pointers (pageable or pinned), split the batch into 32,768-element chunks and
 * overlap each chunk's H2D copy, kernels and D2H copy with the host-side copy of the previous
 * chunk on two internal streams of the current device.  They block until the host output is
 * complete.  Scratch (pinned staging, device buffers) is per device and reused across calls;
 * calls on one device are serialised.  Results are bit-identical to the device-buffer calls. */

/* ①–④: x_host float32 [n_values] -> quantise + pack (codec) -> encrypt (key-holder CRT path when
 * priv is non-NULL, else the public path; r from Philox(seed, ctr0 + plaintext index)) ->
 * c_host [ceil(n_values/slots)][ct_words].  Errors: FLB_EINVAL, FLB_ECUDA, as the batch calls. */
int flb_pack_encrypt_host(const flb_pub* pub, const flb_priv* priv, const flb_codec* codec,
                          const float* x_host, size_t n_values, uint64_t seed, uint64_t ctr0,
                          uint32_t* c_host);

/* ①–④ for several value arrays at once (e.g. the gradients of several clients): array a is packed
 * into its own ceil(n_values[a]/slots) plaintexts (its own slot alignment) and all plaintexts are
 * encrypted as one batch, in array order, with counter ctr0 + global plaintext index; c_host
 * receives sum_a ceil(n_values[a]/slots) ciphertexts.  Same bits as one flb_pack_encrypt_host call
 * per array with the matching ctr0. */
int flb_pack_encrypt_host_multi(const flb_pub* pub, const flb_priv* priv, const flb_codec* codec,
                                const float* const* x_hosts, const size_t* n_values, size_t n_arrays,
                                uint64_t seed, uint64_t ctr0, uint32_t* c_host);

/* ⑤–⑨: c_host [ceil(n_values/slots)][ct_words] -> decrypt -> unpack + dequantise -> x_host
 * float32 [n_values]; summands_host: uint32 [ceil(n_values/slots)] or NULL (then
 * summands_scalar).  pub must be priv's public key.  Errors: FLB_EINVAL, FLB_ECUDA. */
int flb_decrypt_unpack_host(const flb_priv* priv, const flb_pub* pub, const flb_codec* codec,
                            const uint32_t* c_host, size_t n_values, const uint32_t* summands_host,
                            uint32_t summands_scalar, float* x_host);

/* ④⑤ homomorphic aggregation: flb_reduce_segments over host buffers (c_host
 * [num_inputs][ct_words], idx_host/offsets_host int64, out_host [num_segments][ct_words]). */
int flb_reduce_segments_host(const flb_pub* pub, const uint32_t* c_host, size_t num_inputs,
                             const int64_t* idx_host, const int64_t* offsets_host,
                             size_t num_segments, size_t max_segment_len, uint32_t* out_host);

/* Debug entry for the Montgomery primitive (PAPER Alg. 2): out_i = a_i b_i R^-1
 * mod n^2, R = 2^(32 ct_words), canonical.  a_i < n^2, b_i < n^2.  [count][ct_words]. */
int flb_debug_mont_mul(const flb_pub* pub, const uint32_t* a, const uint32_t* b, uint32_t* out,
                       size_t count, void* stream);

/* Debug: the plain product phase of the tensor-core Montgomery kernel (csrc/flb_tc.cuh): t_i = a_i b_i
 * (square != 0: a_i^2, b ignored but must be valid) as 2 words-limb integers, for count <= 128
 * elements of words in {32, 64, 96, 128} limbs.  a, b: [count][words], t: [count][2 words], device.
 * Errors: FLB_EINVAL. */
int flb_debug_tc_product(const uint32_t* a, const uint32_t* b, uint32_t* t, uint32_t count, uint32_t words,
                         int square, void* stream);

/* Algorithmic cost of one element of an op, for roofline accounting: *mont_muls = Montgomery
 * multiplications the kernel performs per element (window table, schedule, domain entry/exit),
 * *limb_products = their CIOS limb-product count (2s^2 + s per s-limb multiplication, s^2 for
 * the plain low-half product of the exact division).  op: 0 = encrypt (pub), 1 = decrypt
 * (priv), 2 = add (pub), 3 = one reduce input (pub; excludes the per-chunk fix-up),
 * 4 = key-holder encrypt (priv); for the tensor-core kernels (k_tc_exp: Montgomery reduction as
 * u8 MMAs, PAPER Alg. 1 L98-L114 restated as a contraction against the shared modulus), whose IMAD
 * work is only the S^2 limb products of t = a b per S-word multiplication: 5 = key-holder encrypt
 * (both stages, priv), 6 = decrypt's two exponentiations (priv); *limb_products = those
 * products on the IMAD pipe (S^2 per product, S (S + 1) / 2 per block squaring);
 * 7 / 8 = the same two ops with *limb_products = their u8 MMA MACs (2 (4S)^2 per product).
 * Host only.  Errors: FLB_EINVAL; FLB_EUNSUPPORTED for ops 5/6 on keys without the path. */
int flb_op_cost(const flb_pub* pub, const flb_priv* priv, int op, uint64_t* mont_muls,
                uint64_t* limb_products);

/* Thread-local description of the last non-OK status ("" if none). */
const char* flb_last_error(void);

/* Library version string. */
const char* flb_version(void);

#ifdef __cplusplus
}
#endif

#endif /* FLB_PAILLIER_H */
