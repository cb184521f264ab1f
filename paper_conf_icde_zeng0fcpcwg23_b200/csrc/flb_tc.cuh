// flb_tc.cuh — Montgomery multiplication with the reduction on the 5th-generation tensor cores.
//
// Every element of a Paillier batch shares its modulus N (n^2, p^2 or q^2), so the reduction half
// of a Montgomery product c = a b R^-1 mod N (PAPER Alg. 1, L98–L114: q = t N' mod R, then
// (t + q N) / R) is a dense contraction of the whole batch against two constant matrices:
//   q   = t_lo * N'  mod R       (t_lo: the low S words of t = a b; N' = -N^-1 mod R)
//   u   = (t + q N) / R
// Written over bytes, t_lo * N' is a convolution, i.e. the product of the batch's byte rows with a
// Toeplitz matrix of N' bytes, and the same for q N: u8 x u8 products summed in s32 (< 2^24, exact)
// by `tcgen05.mma.kind::i8` with the accumulators in TMEM.  Only the plain product t = a b (S^2
// limb products, half of CIOS's 2 S^2) stays on the integer pipe.  The result is the canonical
// Montgomery product, bit-identical to mont_mul (flb_bn.cuh).
//
// Tile: 128 elements per CTA (one per TMEM lane / MMA row), 512 threads.  Per multiplication:
//   P   all 16 warps: groups of T = 4 lanes compute t = a b (row-scanning product, X = S/4 limbs
//       per lane); t_lo goes to the MMA operand tile sA as bytes, t_hi to the element's work row;
//   M1  one thread: D1[128 x 4S] = sA x B1 (B1[n][k] = N'_(n-k) bytes, n, k < 4S);
//   N1  warps 0-3 (thread i = element i = TMEM lane i): carry-normalise D1's row into q mod R,
//       written over sA;
//   M2  one thread: D2 = sA x B2 for output byte columns 4S-16 .. 8S-1 (B2 = Toeplitz of N bytes);
//   F   warps 0-3: u = t_hi + high(q N) + c', where the carry c' out of the low half is exact from
//       the top 16 low columns alone (t_lo + (q N mod R) is a multiple of R; see stage F in tc_mont), then
//       one conditional subtraction (u < 2N); u is written to the element's work row.
#pragma once
#include <cstdint>
#include "flb_kernels.cuh"  // flb_bn.cuh + the group load/store helpers

namespace flb {
namespace tc {

constexpr int kTileM = 128;     // elements per CTA tile (MMA M, TMEM lanes)
constexpr int kThreads = 512;   // 16 warps
constexpr int kT = 4;           // lanes per element in the product phase
constexpr int kBoundary = 16;   // low columns of q N read for the carry into the high half

template <int S>
struct Cfg {
  static constexpr int X = S / kT;                 // limbs per lane
  static constexpr int KB = 4 * S;                 // bytes of an S-word operand (MMA K and N)
  static constexpr int KCH = KB / 16;              // 16-byte chunks per operand row
  static constexpr int LD = X + 4;                 // staged multiplier row (words)
  static constexpr int W0 = S + 16 > kT * LD ? S + 16 : kT * LD;
  static constexpr int WROW = ((W0 + 3) / 4) % 2 == 0 ? ((W0 + 3) / 4) * 4 + 4 : ((W0 + 3) / 4) * 4;  // /4 odd
  static constexpr int TMEM_COLS = 2 * KB <= 256 ? 256 : 512;
  static constexpr int D2H_COL = KB;               // TMEM column of the high half of q N
  // dynamic shared memory carve-up (bytes)
  static constexpr int OFF_B1 = 0;
  static constexpr int OFF_B2H = OFF_B1 + KB * KB;
  static constexpr int OFF_B2B = OFF_B2H + KB * KB;
  static constexpr int OFF_A = OFF_B2B + kBoundary * KB;
  static constexpr int OFF_W = OFF_A + kTileM * KB;
  static constexpr int OFF_X = OFF_W + kTileM * WROW * 4;  // carry exchange, 4 x uint4 per element
  static constexpr int SMEM = OFF_X + kTileM * 4 * 16;
  static_assert(KB <= 256, "one MMA covers N <= 256 output columns");
  static_assert(X % 4 == 0, "16-byte limb chunks");
};

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

// byte offset of (row, k) in the K-major no-swizzle core-matrix layout (8 rows x 16 bytes per core
// matrix, K chunks 128 B apart = LBO, 8-row groups kch * 128 B apart = SBO)
__host__ __device__ __forceinline__ uint32_t cm_off(uint32_t row, uint32_t k, uint32_t kch) {
  return (row >> 3) * (kch * 128u) + (k >> 4) * 128u + (row & 7u) * 16u + (k & 15u);
}

__device__ __forceinline__ uint64_t smem_desc(uint32_t saddr, uint32_t sbo) {
  uint64_t d = (uint64_t)((saddr & 0x3FFFFu) >> 4);
  d |= (uint64_t)(128u >> 4) << 16;                 // LBO: next 16-byte K chunk
  d |= (uint64_t)((sbo >> 4) & 0x3FFFu) << 32;      // SBO: next 8-row group
  d |= (uint64_t)1 << 46;                           // descriptor version (sm_100)
  return d;                                         // SWIZZLE_NONE, base offset 0
}

// kind::i8 instruction descriptor: s32 accumulator, u8 x u8, both K-major
__device__ __forceinline__ uint32_t idesc_u8(int m, int n) {
  return (2u << 4) | ((uint32_t)(n >> 3) << 17) | ((uint32_t)(m >> 4) << 24);
}

// D[tmem] (+)= A[128 x 32k..] x B[n x 32k..]^T over kch/2 K-slices of 32 bytes
__device__ __forceinline__ void mma_u8(uint32_t tmem_d, uint32_t sa, uint32_t sb, uint32_t kch, uint32_t idesc) {
  for (uint32_t ks = 0; ks < kch / 2; ks++) {
    const uint64_t ad = smem_desc(sa + ks * 256u, kch * 128u);
    const uint64_t bd = smem_desc(sb + ks * 256u, kch * 128u);
    const uint32_t acc = ks > 0 ? 1u : 0u;
    asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
                 "tcgen05.mma.cta_group::1.kind::i8 [%0], %1, %2, %3, p;\n\t}"
                 :: "r"(tmem_d), "l"(ad), "l"(bd), "r"(idesc), "r"(acc));
  }
}

__device__ __forceinline__ void mma_commit(uint64_t* mbar) {
  asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" :: "r"(smem_u32(mbar)));
}

__device__ __forceinline__ void mbar_wait(uint64_t* mbar, uint32_t phase) {
  asm volatile("{\n\t.reg .pred P1;\n\tWAIT_%=:\n\t"
               "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n\t"
               "@!P1 bra WAIT_%=;\n\t}" :: "r"(smem_u32(mbar)), "r"(phase));
}

__device__ __forceinline__ void fence_async_smem() { asm volatile("fence.proxy.async.shared::cta;" ::: "memory"); }
__device__ __forceinline__ void tc_before_sync() { asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void tc_after_sync() { asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory"); }

// 32 consecutive s32 columns of this thread's TMEM lane (warp w owns lanes 32w .. 32w+31)
__device__ __forceinline__ void tmem_ld32(uint32_t taddr, uint32_t (&v)[32]) {
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x32.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,"
      "%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%32];"
      : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7]),
        "=r"(v[8]), "=r"(v[9]), "=r"(v[10]), "=r"(v[11]), "=r"(v[12]), "=r"(v[13]), "=r"(v[14]), "=r"(v[15]),
        "=r"(v[16]), "=r"(v[17]), "=r"(v[18]), "=r"(v[19]), "=r"(v[20]), "=r"(v[21]), "=r"(v[22]), "=r"(v[23]),
        "=r"(v[24]), "=r"(v[25]), "=r"(v[26]), "=r"(v[27]), "=r"(v[28]), "=r"(v[29]), "=r"(v[30]), "=r"(v[31])
      : "r"(taddr));
  asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
}

__device__ __forceinline__ void tmem_ld16(uint32_t taddr, uint32_t (&v)[16]) {
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
      : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7]),
        "=r"(v[8]), "=r"(v[9]), "=r"(v[10]), "=r"(v[11]), "=r"(v[12]), "=r"(v[13]), "=r"(v[14]), "=r"(v[15])
      : "r"(taddr));
  asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
}

// four byte-column sums (each < 2^25) as one 32-bit-word contribution, plus a carry and an addend
__device__ __forceinline__ uint64_t word_of(uint32_t c0, uint32_t c1, uint32_t c2, uint32_t c3) {
  return (uint64_t)c0 + ((uint64_t)c1 << 8) + ((uint64_t)c2 << 16) + ((uint64_t)c3 << 24);
}

struct Smem {
  uint8_t* base;
  uint32_t tmem;
  uint64_t* mbar;
};

#ifndef FLB_TC_PROF
#define FLB_TC_PROF 0
#endif
#if FLB_TC_PROF
// per-phase cycle totals of thread 0 (P, M1 wait, N1, M2 wait, F, calls): FLB_TC_PROF=1 builds only
static __device__ unsigned long long g_tc_prof[8];
#define TC_MARK(slot)                                              \
  do {                                                             \
    if (threadIdx.x == 0) {                                        \
      const long long now_ = clock64();                            \
      atomicAdd(&g_tc_prof[slot], (unsigned long long)(now_ - t_)); \
      t_ = now_;                                                   \
    }                                                              \
  } while (0)
#else
#define TC_MARK(slot) do {} while (0)
#endif

// Montgomery product of the tile: this group's element has a, b in registers (X limbs per lane);
// on return the canonical a b R^-1 mod N is in the element's work row (words 0..S-1).  `phase`
// tracks the mbarrier parity (two completions per call).  Collective over the whole CTA.
template <int S>
__device__ __forceinline__ void tc_mont(const uint32_t (&a)[Cfg<S>::X], const uint32_t (&b)[Cfg<S>::X],
                                        const Smem& sm, const uint32_t* __restrict__ Nmod, uint32_t& phase) {
  using C = Cfg<S>;
  constexpr int X = C::X, LD = C::LD, KCH = C::KCH, KB = C::KB;
  const int tid = threadIdx.x, elem = tid / kT, k = tid % kT, warp = tid >> 5;
  uint8_t* sA = sm.base + C::OFF_A;
  uint32_t* sW = reinterpret_cast<uint32_t*>(sm.base + C::OFF_W);
  uint32_t* grp = sW + elem * C::WROW;
#if FLB_TC_PROF
  long long t_ = clock64();
#endif
  // ---- P: t = a b (rows of b's words staged in the element's work row)
  {
    __syncwarp();
    uint4* q = reinterpret_cast<uint4*>(grp + k * LD);
#pragma unroll
    for (int v = 0; v < X / 4; v++) q[v] = make_uint4(b[4 * v], b[4 * v + 1], b[4 * v + 2], b[4 * v + 3]);
    __syncwarp();
    uint32_t E[X + 1], O[X + 1], pend = 0, lo[X], hi[X];
    const uint32_t dummy[X] = {};
#pragma unroll
    for (int t = 0; t <= X; t++) { E[t] = 0; O[t] = 0; }
#pragma unroll
    for (int t = 0; t < X; t++) lo[t] = 0;
#pragma unroll 1
    for (int kk = 0; kk < kT; kk++) {
      const uint32_t* row = grp + kk * LD;
#pragma unroll
      for (int jj = 0; jj < X; jj++) {
        const uint32_t w = cios_step<X, kT, false>(E, O, pend, a, row[jj], dummy, 0u);
        if (k == kk) lo[jj] = w;
      }
    }
    collapse<X, kT>(hi, E, O, pend);
    __syncwarp();
#pragma unroll
    for (int v = 0; v < X / 4; v++) {
      *reinterpret_cast<uint4*>(sA + cm_off(elem, 16u * (k * X / 4 + v), KCH)) =
          make_uint4(lo[4 * v], lo[4 * v + 1], lo[4 * v + 2], lo[4 * v + 3]);
      *reinterpret_cast<uint4*>(grp + k * X + 4 * v) = make_uint4(hi[4 * v], hi[4 * v + 1], hi[4 * v + 2], hi[4 * v + 3]);
    }
    fence_async_smem();
  }
  tc_before_sync();
  __syncthreads();
  TC_MARK(0);
  // ---- M1: q columns
  if (tid == 0) {
    tc_after_sync();
    mma_u8(sm.tmem, smem_u32(sA), smem_u32(sm.base + C::OFF_B1), KCH, idesc_u8(kTileM, KB));
    mma_commit(sm.mbar);
  }
  // every warp normalises: TMEM lane quadrant L = warp % 4 (elements 32L .. 32L+31), column quarter
  // g = warp / 4 (QW words = QC byte columns); carries cross quarters through `xch` (exact)
  constexpr int QW = S / 4, QC = 4 * QW;
  const int L = warp & 3, g = warp >> 2, i = 32 * L + (tid & 31);
  const uint32_t lane_base = sm.tmem + ((uint32_t)(32 * L) << 16);
  uint32_t* row = sW + i * C::WROW;
  uint4* xch = reinterpret_cast<uint4*>(sm.base + C::OFF_X) + i * 4;
  uint4 ttop = make_uint4(0, 0, 0, 0);
  if (g == 0) ttop = *reinterpret_cast<const uint4*>(sA + cm_off(i, KB - 16, KCH));  // t_lo top 16 bytes
  mbar_wait(sm.mbar, phase);
  phase ^= 1u;
  tc_after_sync();
  TC_MARK(1);
  uint32_t v[QW];
  // carry into this quarter from the quarters below: cin_{h+1} = C_h + [word0_h + cin_h overflows
  // and words 1.. of quarter h are all ones]; returns the carry out of quarter `upto` - 1
  auto resolve = [&](int upto) {
    uint64_t cin = 0;
    for (int h = 0; h < upto; h++) {
      const uint4 x = xch[h];
      const uint64_t ov = (x.z != 0u && (((uint64_t)x.y + cin) >> 32) != 0) ? 1u : 0u;
      cin = (uint64_t)x.x + ov;
    }
    return cin;
  };
  auto add_in = [&](uint64_t cin) {
#pragma unroll
    for (int w = 0; w < QW; w++) {
      const uint64_t s = (uint64_t)v[w] + cin;
      v[w] = (uint32_t)s;
      cin = s >> 32;
    }
  };
  // ---- N1: q = D1 mod R (quarter g, local carry chain), bytes back into sA
  {
    uint64_t carry = 0;
#pragma unroll
    for (int c0 = 0; c0 < QC; c0 += 32) {
      uint32_t cv[32];
      tmem_ld32(lane_base + (uint32_t)(g * QC + c0), cv);
#pragma unroll
      for (int w = 0; w < 8; w++) {
        const uint64_t s = carry + word_of(cv[4 * w], cv[4 * w + 1], cv[4 * w + 2], cv[4 * w + 3]);
        v[c0 / 4 + w] = (uint32_t)s;
        carry = s >> 32;
      }
    }
    uint32_t ao = 0xffffffffu;
#pragma unroll
    for (int w = 1; w < QW; w++) ao &= v[w];
    xch[g] = make_uint4((uint32_t)carry, v[0], ao == 0xffffffffu ? 1u : 0u, 0u);
  }
  tc_before_sync();
  __syncthreads();  // all D1 reads and all t_lo reads of sA done; carries published
  add_in(resolve(g));
#pragma unroll
  for (int c = 0; c < QW / 4; c++)
    *reinterpret_cast<uint4*>(sA + cm_off(i, g * QC + 16 * c, KCH)) = make_uint4(v[4 * c], v[4 * c + 1], v[4 * c + 2], v[4 * c + 3]);
  fence_async_smem();
  tc_before_sync();
  __syncthreads();
  // ---- M2: q N, columns 4S-16 .. 8S-1
  if (tid == 0) {
    tc_after_sync();
    mma_u8(sm.tmem + C::D2H_COL, smem_u32(sA), smem_u32(sm.base + C::OFF_B2H), KCH, idesc_u8(kTileM, KB));
    mma_u8(sm.tmem, smem_u32(sA), smem_u32(sm.base + C::OFF_B2B), KCH, idesc_u8(kTileM, kBoundary));
    mma_commit(sm.mbar);
  }
  TC_MARK(2);
  mbar_wait(sm.mbar, phase);
  phase ^= 1u;
  tc_after_sync();
  TC_MARK(3);
  // ---- F: u = t_hi + high(q N) + c'.  The carry out of the low half: t_lo + (q N mod R) = c' R
  // exactly; with W = the top 16 low byte columns of t + q N (as an integer over those columns) and
  // Z the rest (< 2^(8(4S-16)+26)), c' R = W 2^(8(4S-16)) + Z, so c' = ceil(W / 2^128): the floor
  // plus one when W mod 2^128 != 0.  Quarter 0 starts its chain with c'.
  {
    uint64_t carry = 0;
    if (g == 0) {
      uint32_t bc[16];
      tmem_ld16(lane_base, bc);
      const uint32_t tt[4] = {ttop.x, ttop.y, ttop.z, ttop.w};
      uint32_t nz = 0;
#pragma unroll
      for (int w = 0; w < 4; w++) {
        const uint64_t s = carry + word_of(bc[4 * w], bc[4 * w + 1], bc[4 * w + 2], bc[4 * w + 3]) + tt[w];
        nz |= (uint32_t)s;
        carry = s >> 32;
      }
      carry += nz != 0u ? 1u : 0u;
    }
#pragma unroll
    for (int c0 = 0; c0 < QC; c0 += 32) {
      uint32_t cv[32];
      tmem_ld32(lane_base + (uint32_t)(C::D2H_COL + g * QC + c0), cv);
      const uint4 h0 = reinterpret_cast<const uint4*>(row + g * QW + c0 / 4)[0];
      const uint4 h1 = reinterpret_cast<const uint4*>(row + g * QW + c0 / 4)[1];
      const uint32_t th[8] = {h0.x, h0.y, h0.z, h0.w, h1.x, h1.y, h1.z, h1.w};
#pragma unroll
      for (int w = 0; w < 8; w++) {
        const uint64_t s = carry + word_of(cv[4 * w], cv[4 * w + 1], cv[4 * w + 2], cv[4 * w + 3]) + th[w];
        v[c0 / 4 + w] = (uint32_t)s;
        carry = s >> 32;
      }
    }
    uint32_t ao = 0xffffffffu;
#pragma unroll
    for (int w = 1; w < QW; w++) ao &= v[w];
    xch[g] = make_uint4((uint32_t)carry, v[0], ao == 0xffffffffu ? 1u : 0u, 0u);
  }
  tc_before_sync();
  __syncthreads();
  const uint64_t ovf = resolve(4);  // bit above S words (u < 2N < 2R)
  add_in(resolve(g));
  // u - N over this quarter: local borrow B_g, zero-difference flag Z_g
  uint32_t d[QW];
  {
    uint32_t br = 0, nzd = 0;
#pragma unroll
    for (int c = 0; c < QW / 4; c++) {
      const uint4 nv = __ldg(reinterpret_cast<const uint4*>(Nmod + g * QW + 4 * c));
      const uint32_t nn[4] = {nv.x, nv.y, nv.z, nv.w};
#pragma unroll
      for (int w = 0; w < 4; w++) {
        const uint64_t df = (uint64_t)v[4 * c + w] - nn[w] - br;
        d[4 * c + w] = (uint32_t)df;
        br = (uint32_t)(df >> 63);
        nzd |= (uint32_t)df;
      }
    }
    xch[g].w = br | (nzd == 0u ? 2u : 0u);
  }
  __syncthreads();
  {
    uint32_t bin = 0, bout;
    for (int h = 0; h < 4; h++) {
      if (h == g) bout = bin;  // borrow into this quarter
      const uint32_t f = xch[h].w;
      bin = (f & 1u) | ((f >> 1) & bin);
    }
    const bool take = ovf != 0 || bin == 0;  // u >= N
    if (take) {
      uint32_t br = bout;
#pragma unroll
      for (int w = 0; w < QW; w++) {
        const uint64_t df = (uint64_t)d[w] - br;
        v[w] = (uint32_t)df;
        br = (uint32_t)(df >> 63);
      }
    }
#pragma unroll
    for (int c = 0; c < QW / 4; c++)
      reinterpret_cast<uint4*>(row + g * QW)[c] = make_uint4(v[4 * c], v[4 * c + 1], v[4 * c + 2], v[4 * c + 3]);
  }
  tc_before_sync();
  __syncthreads();
  TC_MARK(4);
#if FLB_TC_PROF
  if (threadIdx.x == 0) atomicAdd(&g_tc_prof[5], 1ull);
#endif
}

// this group's X limbs of the element's work row
template <int S>
__device__ __forceinline__ void tc_row_load(uint32_t (&r)[Cfg<S>::X], const Smem& sm) {
  using C = Cfg<S>;
  const int elem = threadIdx.x / kT, k = threadIdx.x % kT;
  const uint32_t* row = reinterpret_cast<const uint32_t*>(sm.base + C::OFF_W) + elem * C::WROW + k * C::X;
#pragma unroll
  for (int v = 0; v < C::X / 4; v++) {
    const uint4 u = reinterpret_cast<const uint4*>(row)[v];
    r[4 * v] = u.x; r[4 * v + 1] = u.y; r[4 * v + 2] = u.z; r[4 * v + 3] = u.w;
  }
}

}  // namespace tc
}  // namespace flb

namespace flb {
namespace tc {

// ----------------------------------------------------------------------------- key-holder stage 2
// c_P = (1 + m n) y^P mod P^2 for one prime P per launch (Eq. 3 with g = n + 1, by the
// two-stage CRT of k_encrypt_crt2: y = r^Q mod P from k_crt_pre), every Montgomery product by
// tc_mont.  Persistent CTAs over 128-element tiles; the odd-power window table of each element
// lives in global scratch [entry][elem][S] per CTA (entry `table` holds x^2, then the saved power).
struct PowArgs {
  const uint32_t* P2;      // modulus P^2 (S words)
  const uint32_t* R2;      // R^2 mod P^2
  const uint32_t* nR;      // n R mod P^2
  const uint32_t* B1;      // Toeplitz(N') core-matrix operand, KB x KB bytes
  const uint32_t* B2h;     // Toeplitz(N) high columns, KB x KB bytes
  const uint32_t* B2b;     // Toeplitz(N) boundary columns, 16 x KB bytes
  const uint32_t* sched;   // schedule of the exponent P
  int sched_len, table;
  const uint32_t* y;       // [count][H]
  uint32_t H;
  const uint32_t* m;       // [count][S]
  uint32_t* out;           // [count][S]
  uint64_t count;
  uint32_t* scratch;       // gridDim * kTileM * (table + 1) * S words
};

template <int S>
__global__ void __launch_bounds__(kThreads, 1) k_tc_pow(const PowArgs A) {
  using C = Cfg<S>;
  constexpr int X = C::X, KB = C::KB;
  extern __shared__ __align__(1024) uint8_t smem[];
  __shared__ __align__(8) uint64_t mbar;
  __shared__ uint32_t tmem_sh;
  const int tid = threadIdx.x, warp = tid >> 5, elem = tid / kT, k = tid % kT;
  {
    const uint4* s1 = reinterpret_cast<const uint4*>(A.B1);
    const uint4* s2 = reinterpret_cast<const uint4*>(A.B2h);
    const uint4* s3 = reinterpret_cast<const uint4*>(A.B2b);
    uint4* d1 = reinterpret_cast<uint4*>(smem + C::OFF_B1);
    uint4* d2 = reinterpret_cast<uint4*>(smem + C::OFF_B2H);
    uint4* d3 = reinterpret_cast<uint4*>(smem + C::OFF_B2B);
    for (int i = tid; i < KB * KB / 16; i += kThreads) { d1[i] = __ldg(s1 + i); d2[i] = __ldg(s2 + i); }
    for (int i = tid; i < kBoundary * KB / 16; i += kThreads) d3[i] = __ldg(s3 + i);
  }
  if (tid == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" :: "r"(smem_u32(&mbar)));
    asm volatile("fence.mbarrier_init.release.cluster;");
  }
  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" :: "r"(smem_u32(&tmem_sh)),
                 "n"(C::TMEM_COLS));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  fence_async_smem();
  tc_before_sync();
  __syncthreads();
  tc_after_sync();
  const Smem sm{smem, tmem_sh, &mbar};
  uint32_t phase = 0;
  const int TB = A.table;
  uint32_t* tab = A.scratch + (size_t)blockIdx.x * kTileM * (TB + 1) * S;
  auto slot = [&](int ent) { return tab + ((size_t)ent * kTileM + elem) * S + k * X; };
  for (uint64_t tile = blockIdx.x; tile * kTileM < A.count; tile += gridDim.x) {
    const uint64_t e = tile * kTileM + elem;
    const bool valid = e < A.count;
    uint32_t a[X], b[X];
    load_elem<X, kT>(a, A.y + e * A.H, A.H, valid);
    load_const<X, kT>(b, A.R2);
    tc_mont<S>(a, b, sm, A.P2, phase);                     // x = y R mod P^2
    tc_row_load<S>(a, sm);
    store_limbs<X>(slot(0), a);
    if (TB > 1) {
      tc_mont<S>(a, a, sm, A.P2, phase);                   // x^2
      tc_row_load<S>(b, sm);
#pragma unroll 1
      for (int i = 1; i < TB; i++) {
        load_limbs_plain<X>(a, slot(i - 1));
        tc_mont<S>(a, b, sm, A.P2, phase);
        tc_row_load<S>(a, sm);
        store_limbs<X>(slot(i), a);
      }
    }
    const uint32_t op0 = __ldg(A.sched);
    load_limbs_plain<X>(a, slot((int)(op0 >> 16) - 1));
#pragma unroll 1
    for (int o = 1; o < A.sched_len; o++) {
      const uint32_t op = __ldg(A.sched + o);
      const int sq = (int)(op & 0xffffu), idx = (int)(op >> 16) - 1;
#pragma unroll 1
      for (int i = 0; i < sq; i++) {
        tc_mont<S>(a, a, sm, A.P2, phase);
        tc_row_load<S>(a, sm);
      }
      if (idx >= 0) {
        load_limbs_plain<X>(b, slot(idx));
        tc_mont<S>(a, b, sm, A.P2, phase);
        tc_row_load<S>(a, sm);
      }
    }
    store_limbs<X>(slot(TB), a);                           // y^P R
    load_elem<X, kT>(a, A.m + e * S, S, valid);
    load_const<X, kT>(b, A.nR);
    tc_mont<S>(a, b, sm, A.P2, phase);                     // m n mod P^2
    tc_row_load<S>(b, sm);
    {
      uint32_t nn[X];
      load_const<X, kT>(nn, A.P2);
      grp_add_small<X, kT>(b, 1u);
      grp_cond_sub<X, kT>(b, nn, 0u);                      // 1 + m n mod P^2
    }
    load_limbs_plain<X>(a, slot(TB));
    tc_mont<S>(a, b, sm, A.P2, phase);                     // c_P
    tc_row_load<S>(a, sm);
    if (valid) store_limbs<X>(A.out + e * S + k * X, a);
  }
  tc_before_sync();
  __syncthreads();
  if (warp == 0) {
    tc_after_sync();
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" :: "r"(tmem_sh), "n"(C::TMEM_COLS));
  }
}

}  // namespace tc
}  // namespace flb
