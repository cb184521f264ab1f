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
// Tile: 128 elements per CTA (MMA M = 128, one per TMEM lane), 256 threads, two CTAs per SM so the
// warp schedulers overlap one CTA's product phase (integer pipe) with the other's normalisation
// (ALU, TMEM loads, barriers).  Per multiplication (KB = 4S bytes per operand):
//   P   groups of T lanes (X = S/T = 16 limbs each; T = 4 at S = 64 in two passes of 64 elements,
//       T = 2 at S = 32 in one pass of 128) compute t = a b (row-scanning product, the multiplier
//       staged in the element's sA row; squarings at S = 64 by block squaring, tc_square_product);
//       t_lo goes to sA as bytes (the MMA A operand), t_hi to the element's work row;
//   M1  one thread: D1[128 x KB] = sA x B1, B1[n][k] = N'_(n-k) (bytes, k <= n);
//   N1  8 warps (TMEM lane quadrant w % 4, column half w / 4): q = D1 mod R normalised into bytes
//       over sA, the carry between the column halves resolved exactly through shared memory;
//   M2  one thread: D2 = sA x B2 for the byte columns [KB-8, 2KB-8) of q N (one N = KB MMA);
//   F   8 warps: u = t_hi + high(q N) + c' (c' from the 8 columns below KB, the 7 top columns of
//       q N from the top 8 bytes of q and N on the CUDA cores), one conditional subtraction.
// The Toeplitz operands are stored once per K-slice shape: for K-slice ks the B operand is the
// row window starting at KB - 32 ks (B1) or 2KB - 8 - 32 ks (B2) of an extended [rows][32 bytes]
// matrix Ext[r][kk] = V_(r - KB - kk), so B1 and B2 take 2KB x 32 and 3KB x 32 bytes of shared
// memory instead of KB x KB each.
#pragma once
#include <cstdint>
#include "flb_kernels.cuh"  // flb_bn.cuh + the group load/store helpers

namespace flb {
namespace tc {

constexpr int kTileM = 128;     // elements per CTA tile (MMA M, TMEM lanes)
constexpr int kThreads = 256;   // 8 warps; two CTAs per SM (one at S = 128)
constexpr int kT = 4;           // lanes per element in the product phase at S = 64 (S = 32: 2, S = 128: 8)

template <int S>
struct Cfg {
  // lanes per element in the product phase (S = 96, 3072-bit p^2: eight lanes of X = 12 limbs)
  static constexpr int T = S >= 96 ? 8 : S >= 64 ? kT : 2;
  static constexpr int X = S / T;                  // limbs per lane (16; 12 at S = 96)
  // threads per CTA: 8 warps (two CTAs per SM); at S = 128 (one CTA per SM: all TMEM) 16 warps, so
  // the product phase keeps four warps per scheduler
  static constexpr int THREADS = S >= 96 ? 512 : kThreads;
  static constexpr int GW = THREADS / 128;         // warps per TMEM lane quadrant
  static constexpr int EP = THREADS / T;           // elements per product pass
  static constexpr int NP = kTileM / EP;           // product passes per tile
  static constexpr int KB = 4 * S;                 // bytes of an S-word operand (MMA K and N)
  static constexpr int KCH = KB / 16;              // 16-byte chunks per operand row
  // normalisation: each element's byte columns in NG groups, one thread each (the warps of its TMEM
  // lane quadrant): 2 at 256 threads, 4 at S = 128 (512 threads); QW words / QC columns per thread
  static constexpr int NG = THREADS / 128;
  static constexpr int QW = S / NG, QC = KB / NG;
  // work row (t_hi, then the product u): 4 padding words after every 32, so the lanes of one element
  // (16 limbs = 64 bytes each, a quarter of t 128 bytes apart) hit different bank groups; rows
  // WROW words apart with WROW / 4 odd, so 8 consecutive elements do too
  // (S <= 64: unpadded — two CTAs per SM must fit in the SM's 228 KB of shared memory)
  static constexpr int WPAD = S >= 128 ? S + 4 * (S / 32) : S;
  static constexpr int WROW = (WPAD / 4) % 2 == 1 ? WPAD : WPAD + 4;
  // D1 and D2 share TMEM columns [0, KB); the allocation is a power of two (S = 96, 128: all 512)
  static constexpr int TMEM_COLS = KB <= 128 ? 128 : KB <= 256 ? 256 : 512;
  static constexpr int CTAS_PER_SM = S >= 96 ? 1 : 2;  // TMEM and shared memory per tile
  // dynamic shared memory carve-up (bytes)
  static constexpr int OFF_E1 = 0;                          // 2 KB rows x 32 bytes
  static constexpr int OFF_E2 = OFF_E1 + 2 * KB * 32;       // 3 KB rows x 32 bytes
  static constexpr int OFF_A = OFF_E2 + 3 * KB * 32;        // 128 x KB bytes (core matrices)
  static constexpr int OFF_W = OFF_A + kTileM * KB;         // 128 work rows
  static constexpr int OFF_X = OFF_W + kTileM * WROW * 4;   // carry exchange, NG x uint2 per element
  static constexpr int SMEM = OFF_X + kTileM * NG * 8;
  static_assert(SMEM <= 227 * 1024, "shared memory per CTA");
  static_assert(CTAS_PER_SM * (SMEM + 1024 + 64) <= 228 * 1024, "CTAS_PER_SM tiles per SM (1 KB reserved per CTA)");
  static_assert(X % 4 == 0 && QW % 8 == 0 && KB <= 512, "16-byte limb chunks, TMEM columns");
};

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

// byte offset of (row, k) in the K-major no-swizzle core-matrix layout (8 rows x 16 bytes per core
// matrix, K chunks 128 B apart = LBO, 8-row groups kch * 128 B apart = SBO)
__host__ __device__ __forceinline__ uint32_t cm_off(uint32_t row, uint32_t k, uint32_t kch) {
  return (row >> 3) * (kch * 128u) + (k >> 4) * 128u + (row & 7u) * 16u + (k & 15u);
}
// padded position of word w of a work row (S = 128: 4 padding words after every 32; Cfg::WPAD)
template <int S>
__host__ __device__ __forceinline__ int wpad(int w) { return S >= 128 ? w + 4 * (w >> 5) : w; }

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

// One K-slice MMA (A columns 32 ks .., B window starting at extended row r) into D columns [c0, c0 + n);
// one instruction covers N <= 256 columns, so a wider slice (KB = 512 at S = 128) is issued in
// 256-column pieces (the B window and the TMEM columns advance together).  KB is a template
// parameter so the slice loops unroll and every (r, c0, n) is a constant.
template <int KB>
__device__ __forceinline__ void mma_slice(uint32_t tmem_d, uint32_t sa, uint32_t ext, uint32_t ks, uint32_t r,
                                          uint32_t c0, uint32_t n, uint32_t acc) {
  const uint64_t ad = smem_desc(sa + ks * 256u, (uint32_t)KB * 8u);
#pragma unroll
  for (uint32_t o = 0; o < (uint32_t)KB; o += 256u) {
    if (o < n) {
      const uint32_t nn = n - o < 256u ? n - o : 256u;
      const uint64_t bd = smem_desc(ext + ((r + o) >> 3) * 256u, 256u);
      asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
                   "tcgen05.mma.cta_group::1.kind::i8 [%0], %1, %2, %3, p;\n\t}"
                   :: "r"(tmem_d + c0 + o), "l"(ad), "l"(bd), "r"(idesc_u8(128, (int)nn)), "r"(acc));
    }
  }
}

// M1: D[:, j] = sum_K A[:, K] V[j - K] for j < KB (the low half of a Toeplitz product, V = N').
// Slice ks (K in [32 ks, 32 ks + 32)) adds nothing to the columns j < 32 ks, so it is issued for
// columns [32 ks, KB) only (its B window then starts at extended row KB for every ks): 36/64 of the
// full MACs.  Slice 0 (all columns) initialises D.
template <int KB>
__device__ __forceinline__ void mma_toeplitz_lo(uint32_t tmem_d, uint32_t sa, uint32_t ext) {
#pragma unroll
  for (uint32_t ks = 0; ks < (uint32_t)KB / 32u; ks++)
    mma_slice<KB>(tmem_d, sa, ext, ks, KB, 32u * ks, KB - 32u * ks, ks > 0);
}
// M2: D[:, j] = sum_K A[:, K] V[KB - 8 + j - K] (V = N, zero at index >= KB) for j < KB: slice ks
// reaches only the columns j < 32 ks + 40, so it is issued for [0, min(KB, 32 ks + 48)); the widest
// slice goes first and initialises D.
template <int KB>
__device__ __forceinline__ void mma_toeplitz_hi(uint32_t tmem_d, uint32_t sa, uint32_t ext) {
#pragma unroll
  for (int ks = KB / 32 - 1; ks >= 0; ks--) {
    const uint32_t n = min((uint32_t)KB, 32u * (uint32_t)ks + 48u);
    mma_slice<KB>(tmem_d, sa, ext, (uint32_t)ks, 2u * KB - 8u - 32u * (uint32_t)ks, 0u, n, ks != KB / 32 - 1);
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

// consecutive s32 columns of this thread's TMEM lane (warp w owns lanes 32 (w % 4) ..)
__device__ __forceinline__ void tmem_ld32(uint32_t taddr, uint32_t* v) {
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x32.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,"
      "%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%32];"
      : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7]),
        "=r"(v[8]), "=r"(v[9]), "=r"(v[10]), "=r"(v[11]), "=r"(v[12]), "=r"(v[13]), "=r"(v[14]), "=r"(v[15]),
        "=r"(v[16]), "=r"(v[17]), "=r"(v[18]), "=r"(v[19]), "=r"(v[20]), "=r"(v[21]), "=r"(v[22]), "=r"(v[23]),
        "=r"(v[24]), "=r"(v[25]), "=r"(v[26]), "=r"(v[27]), "=r"(v[28]), "=r"(v[29]), "=r"(v[30]), "=r"(v[31])
      : "r"(taddr));
}
__device__ __forceinline__ void tmem_ld16(uint32_t taddr, uint32_t* v) {
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
      : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7]),
        "=r"(v[8]), "=r"(v[9]), "=r"(v[10]), "=r"(v[11]), "=r"(v[12]), "=r"(v[13]), "=r"(v[14]), "=r"(v[15])
      : "r"(taddr));
}
__device__ __forceinline__ void tmem_ld8(uint32_t taddr, uint32_t* v) {
  asm volatile("tcgen05.ld.sync.aligned.32x32b.x8.b32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
               : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7])
               : "r"(taddr));
}
__device__ __forceinline__ void tmem_wait() { asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory"); }

// carry-flag chains (one IADD3(.X) per word; the flag lives between consecutive asm statements,
// which no other instruction of this file touches)
__device__ __forceinline__ uint32_t add_cc(uint32_t a, uint32_t b) {
  uint32_t r;
  asm volatile("add.cc.u32 %0, %1, %2;" : "=r"(r) : "r"(a), "r"(b));
  return r;
}
__device__ __forceinline__ uint32_t addc_cc(uint32_t a, uint32_t b) {
  uint32_t r;
  asm volatile("addc.cc.u32 %0, %1, %2;" : "=r"(r) : "r"(a), "r"(b));
  return r;
}
__device__ __forceinline__ uint32_t addc_end(uint32_t a, uint32_t b) {
  uint32_t r;
  asm volatile("addc.u32 %0, %1, %2;" : "=r"(r) : "r"(a), "r"(b));
  return r;
}
__device__ __forceinline__ uint32_t sub_cc(uint32_t a, uint32_t b) {
  uint32_t r;
  asm volatile("sub.cc.u32 %0, %1, %2;" : "=r"(r) : "r"(a), "r"(b));
  return r;
}
__device__ __forceinline__ uint32_t subc_cc(uint32_t a, uint32_t b) {
  uint32_t r;
  asm volatile("subc.cc.u32 %0, %1, %2;" : "=r"(r) : "r"(a), "r"(b));
  return r;
}
__device__ __forceinline__ uint32_t subc_end(uint32_t a, uint32_t b) {
  uint32_t r;
  asm volatile("subc.u32 %0, %1, %2;" : "=r"(r) : "r"(a), "r"(b));
  return r;
}

// Normalise 8 words of byte-column sums c_j (each < 2^25; j = 4w + r) plus optional addends th_w
// into v[0..8), entirely on the integer ALU pipe (the FMA-heavy pipe carries the limb products).
// sum_j c_j 2^(8j) = C_0 + 2^8 C_1 + 2^16 C_2 + 2^24 C_3 with C_r = sum_w c_(4w+r) 2^(32w): word w of
// 2^(8r) C_r is the funnel shift of c_(4w+r) with the previous word's c_(4w-4+r) (its bits above
// 2^32 spill into word w + 1), so word w of the sum is the 64-bit S_w = c_4w + f1_w + f2_w + f3_w
// (+ th_w) (IADD3 pairs, off the carry chain) and v_w = lo S_w + hi S_(w-1) + flag (one addc.cc
// per word).  State across chunks: the last columns of residues 1..3 (p1..p3) and hi S of the last
// word (hprev).  first: the chain starts here (add.cc).
struct NormState {
  uint32_t p1 = 0, p2 = 0, p3 = 0, hprev = 0;
  // everything above the normalised words: the final flag + hi S of the last word + the spills of
  // the last word's shifted columns
  __device__ __forceinline__ uint32_t carry_out_end() {
    return addc_end(hprev, 0u) + (p1 >> 24) + (p2 >> 16) + (p3 >> 8);
  }
};
template <bool TH>
__device__ __forceinline__ void norm8_chain(const uint32_t (&cv)[32], const uint32_t* th, uint32_t* v, NormState& st,
                                            bool first) {
  uint32_t lo[8], hi[8];
  uint32_t p1 = st.p1, p2 = st.p2, p3 = st.p3;
#pragma unroll
  for (int w = 0; w < 8; w++) {
    const uint32_t f1 = __funnelshift_l(p1, cv[4 * w + 1], 8);
    const uint32_t f2 = __funnelshift_l(p2, cv[4 * w + 2], 16);
    const uint32_t f3 = __funnelshift_l(p3, cv[4 * w + 3], 24);
    p1 = cv[4 * w + 1];
    p2 = cv[4 * w + 2];
    p3 = cv[4 * w + 3];
    uint64_t S = (uint64_t)cv[4 * w] + f1 + f2;
    S += TH ? (uint64_t)f3 + th[w] : (uint64_t)f3;
    lo[w] = (uint32_t)S;
    hi[w] = (uint32_t)(S >> 32);
  }
  st.p1 = p1;
  st.p2 = p2;
  st.p3 = p3;
  v[0] = first ? add_cc(lo[0], st.hprev) : addc_cc(lo[0], st.hprev);
#pragma unroll
  for (int w = 1; w < 8; w++) v[w] = addc_cc(lo[w], hi[w - 1]);
  st.hprev = hi[7];
}

// np: product passes of the current unit (Cfg::NP for a whole tile, 1 for a half unit: k_tc_exp)
struct Smem {
  uint8_t* base;
  uint32_t tmem;
  uint64_t* mbar;
  int np;
};

// Half units (k_tc_exp's last, incomplete round of tiles): 64 elements on the rows of product pass 0,
// rows r with r % 32 < 16 (prod_elem); element index of row r of a half unit, relative to its first
// element.  Whole tiles: the identity.
__device__ __forceinline__ int unit_index(int row, bool half) { return half ? ((row >> 5) << 4) + (row & 15) : row; }

// An operand of tc_mont per element of the tile: the element's work row (row = true), or element j
// of an array at p + j * stride with `words` limbs (the rest zero; elements >= `valid` read zeros;
// stride 0 = one constant for all).  `ld` says how the array may be read:
//   kLdNC   ld.global.nc — kernel inputs and key constants, read-only for the whole launch;
//   kLdCTA  plain ld.global — written earlier in the launch by this CTA and ordered by bar.sync
//           (the window-table slots);
//   kLdGPU  ld.relaxed.gpu — written by another CTA of this launch and published by the
//           st.release / ld.acquire tile flag (stage-2 inputs of k_tc_exp_dag).
enum : uint32_t { kLdNC = 0, kLdCTA = 1, kLdGPU = 2 };
struct Src {
  const uint32_t* p;
  uint32_t stride, words, valid;
  bool row;
  uint32_t ld;
  bool half;  // rows map to the elements of a half unit (unit_index)
};
__device__ __forceinline__ Src src_row() { return Src{nullptr, 0, 0, 0, true, kLdNC, false}; }
__device__ __forceinline__ Src src_arr(const uint32_t* p, uint32_t stride, uint32_t words, uint32_t valid,
                                       uint32_t ld = kLdNC, bool half = false) {
  return Src{p, stride, words, valid, false, ld, half};
}

__device__ __forceinline__ uint4 ld_v4(const uint32_t* p, uint32_t ld) {
  uint4 u;
  if (ld == kLdGPU)
    asm volatile("ld.relaxed.gpu.global.v4.u32 {%0,%1,%2,%3}, [%4];"
                 : "=r"(u.x), "=r"(u.y), "=r"(u.z), "=r"(u.w) : "l"(p) : "memory");
  else if (ld == kLdCTA)
    u = *reinterpret_cast<const uint4*>(p);
  else
    u = __ldg(reinterpret_cast<const uint4*>(p));
  return u;
}
__device__ __forceinline__ uint32_t ld_u32(const uint32_t* p, uint32_t ld) {
  uint32_t v;
  if (ld == kLdGPU)
    asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  else if (ld == kLdCTA)
    v = *p;
  else
    v = __ldg(p);
  return v;
}

#ifndef FLB_TC_PROF
#define FLB_TC_PROF 0
#endif
#if FLB_TC_PROF
// per-phase cycle totals of thread 0 (P, M1 wait, N1, M2 wait, F, calls), slots [0, 8) for S = 32
// and [8, 16) for S = 64: FLB_TC_PROF=1 builds only
static __device__ unsigned long long g_tc_prof[16];
#define TC_MARK(slot)                                                                   \
  do {                                                                                  \
    if (threadIdx.x == 0) {                                                             \
      const long long now_ = clock64();                                                 \
      atomicAdd(&g_tc_prof[(S == 64 ? 8 : 0) + (slot)], (unsigned long long)(now_ - t_)); \
      t_ = now_;                                                                        \
    }                                                                                   \
  } while (0)
#else
#define TC_MARK(slot) do {} while (0)
#endif

template <int S>
__device__ __forceinline__ void src_load(uint32_t (&r)[Cfg<S>::X], const Src& s, int elem, const uint32_t* sW) {
  using C = Cfg<S>;
  const int k = threadIdx.x % C::T;
  if (s.row) {
    const uint4* q = reinterpret_cast<const uint4*>(sW + elem * C::WROW + wpad<S>(k * C::X));
#pragma unroll
    for (int v = 0; v < C::X / 4; v++) {
      const uint4 u = q[v];
      r[4 * v] = u.x; r[4 * v + 1] = u.y; r[4 * v + 2] = u.z; r[4 * v + 3] = u.w;
    }
  } else {
    // limbs [k X, k X + X) of the element (the rest of a short element reads zeros)
    const int j = unit_index(elem, s.half);
    const uint32_t* base = s.p + (size_t)j * s.stride;
    const uint32_t w0 = (uint32_t)(k * C::X);
    const bool valid = (uint32_t)j < s.valid;
    if (valid && w0 + C::X <= s.words) {
#pragma unroll
      for (int v = 0; v < C::X / 4; v++) {
        const uint4 u = ld_v4(base + w0 + 4 * v, s.ld);
        r[4 * v] = u.x; r[4 * v + 1] = u.y; r[4 * v + 2] = u.z; r[4 * v + 3] = u.w;
      }
    } else {
#pragma unroll
      for (int j = 0; j < C::X; j++) r[j] = (valid && w0 + j < s.words) ? ld_u32(base + w0 + j, s.ld) : 0u;
    }
  }
}

// Element of the tile that thread tid works on in product pass h (and in the row ops): the warp pair
// (L, L + 4) that normalises elements [32 L, 32 L + 32) in tc_mont also owns them here, so every
// per-element hand-off between phases needs only a barrier over that pair (named barrier 1 + L, 64
// threads); only the MMA issues, which read all 128 rows, need the whole CTA.
template <int S>
__device__ __forceinline__ int prod_elem(int h) {
  constexpr int T = Cfg<S>::T, GW = Cfg<S>::GW;
  const int tid = threadIdx.x, warp = tid >> 5;
  return 32 * (warp & 3) + h * (32 * GW / T) + (warp >> 2) * (32 / T) + (tid & 31) / T;
}
// the warps of TMEM lane quadrant warp % 4 (2 at 256 threads: a warp pair; 4 at 512)
template <int S>
__device__ __forceinline__ void pair_sync() {
  asm volatile("bar.sync %0, %1;" :: "r"(1 + ((threadIdx.x >> 5) & 3)), "n"(32 * Cfg<S>::GW) : "memory");
}

// ----------------------------------------------------------------------------- squaring product
// t = a^2 for the product phase when a = b (87 % of the multiplications of a modexp).  Lane k of the
// element's group holds the limb block a_k = a[kX, kX+X) (X = S/4).  a^2 is the sum of block
// products a_i a_j 2^(32 X (i+j)) over i <= j, the off-diagonal ones doubled; each lane computes
// the same shapes (so the warp never diverges in the multiply code): its diagonal block a_k a_k
// (X x X), one full off-diagonal block a_k a_(k+1 mod 4) (X x X), and half of a_(k&1) a_(k&1)+2
// (X x X/2, row half k>>1): X^2 + X^2 + X^2/2 = 2.5 X^2 = 640 limb products at S = 64 instead of the
// general product's S X = 1024.  Row words of another lane's block arrive by shuffle.  The pieces
// are accumulated in place in t's destination rows (t_lo: the element's sA row, the MMA operand;
// t_hi: its work row) in phases with disjoint word ranges, their carry-outs folded in by one final
// group pass with a ballot carry-lookahead.
template <int X, int R, int W = kT>
__device__ __forceinline__ void blk_prod(uint32_t (&out)[X + R], const uint32_t (&M)[X], const uint32_t (&a)[X],
                                         int src, bool own_upper) {
  // out = M x (R row words of lane src's block): words [0, R) of it by shuffle (every lane serves its
  // own a[j]), or, with own_upper (src is this lane), this lane's words [R, 2R) directly
  uint32_t E[X + 1], O[X + 1], pend = 0;
#pragma unroll
  for (int t = 0; t <= X; t++) { E[t] = 0; O[t] = 0; }
#pragma unroll
  for (int j = 0; j < R; j++) {
    uint32_t bj = __shfl_sync(FULL, a[j], src, W);
    if (R < X && own_upper) bj = a[(j + R) % X];
    out[j] = local_row<X>(E, O, pend, M, bj);
  }
  asm volatile("add.cc.u32 %0, %1, %2;" : "=r"(out[R]) : "r"(E[0]), "r"(pend));
#pragma unroll
  for (int t = 1; t < X; t++) asm volatile("addc.cc.u32 %0, %1, %2;" : "=r"(out[R + t]) : "r"(E[t]), "r"(O[t - 1]));
}

#ifndef FLB_TC_TRISQ
#define FLB_TC_TRISQ 1  // diagonal blocks a_k^2: 1 = one lane-local triangular square, 2 = the half-split form
#endif
#ifndef FLB_TC_TRISQ_S1
#define FLB_TC_TRISQ_S1 1  // stage-1 tiles (S = 32) of k_tc_exp_dag: one triangle (measured with the double-buffered loads)
#endif
#ifndef FLB_TC_TRISQ_S2
#define FLB_TC_TRISQ_S2 1  // stage-2 tiles (S = 64) of k_tc_exp_dag
#endif
#ifndef FLB_TC_TRISQ_EXP
#define FLB_TC_TRISQ_EXP 1  // k_tc_exp (decryption, public, two-launch key-holder stages): one triangle
#endif

// v = a^2 (2X words) for this lane's own block, X (X - 1) / 2 + X limb products instead of X^2
// (squarings dominate the modexp).  U = sum_{i<j} a_i a_j 2^(32 (i + j)) by rows
// j = 0 .. X - 2 (row j: a[j+1, X) x a_j from word 2j + 1), then v = 2 U + sum_i a_i^2 2^(64 i) in
// one carry chain with the doubling as a funnel shift.  Every product is one IMAD.WIDE.U32(.X)
// (ptxas fuses a mad.lo.cc / madc.hi.cc pair into it), whose 64-bit accumulator must be an
// even-aligned register pair: products at even words i + j accumulate into UE (pairs at even
// indices), those at odd words into UO shifted down one word (UO[q] is word q + 1, pairs again at
// even indices), so a row is two carry chains of whole products — i = j+2, j+4, .. into UE and
// i = j+1, j+3, .. into UO — with no register moves; U = UE + 2^32 UO at the end.
// Bounds: UE or UO plus any subset of row j's products is < 2^(32 (X + j + 1)), so a chain that
// ends at word X + j drops its carry and one that ends at X + j - 1 carries into word X + j only.
template <int X, int OFF>
__device__ __forceinline__ void sqr_row_chain(uint32_t (&u)[2 * X], const uint32_t (&a)[X], int j, int i0) {
#pragma unroll
  for (int i = i0; i < X; i += 2) {
    const int p = i + j - OFF;  // accumulator index of the product's low word
    const bool first = i == i0, last = i + 2 >= X;
    const bool top = i + j + 1 == X + j;  // the chain's last word is X + j: no carry out
    if (first && last && top)
      asm volatile("mad.lo.cc.u32 %0, %2, %3, %0;\n\tmadc.hi.u32 %1, %2, %3, %1;"
                   : "+r"(u[p]), "+r"(u[p + 1]) : "r"(a[i]), "r"(a[j]));
    else if (first)
      asm volatile("mad.lo.cc.u32 %0, %2, %3, %0;\n\tmadc.hi.cc.u32 %1, %2, %3, %1;"
                   : "+r"(u[p]), "+r"(u[p + 1]) : "r"(a[i]), "r"(a[j]));
    else if (last && top)
      asm volatile("madc.lo.cc.u32 %0, %2, %3, %0;\n\tmadc.hi.u32 %1, %2, %3, %1;"
                   : "+r"(u[p]), "+r"(u[p + 1]) : "r"(a[i]), "r"(a[j]));
    else
      asm volatile("madc.lo.cc.u32 %0, %2, %3, %0;\n\tmadc.hi.cc.u32 %1, %2, %3, %1;"
                   : "+r"(u[p]), "+r"(u[p + 1]) : "r"(a[i]), "r"(a[j]));
    if (last && !top) asm volatile("addc.u32 %0, %0, 0;" : "+r"(u[X + j - OFF]));
  }
}

template <int X>
__device__ __forceinline__ void sqr_local(uint32_t (&v)[2 * X], const uint32_t (&a)[X]) {
  uint32_t ue[2 * X], uo[2 * X], u[2 * X];
#pragma unroll
  for (int w = 0; w < 2 * X; w++) { ue[w] = 0; uo[w] = 0; }
#pragma unroll
  for (int j = 0; j < X - 1; j++) {
    sqr_row_chain<X, 1>(uo, a, j, j + 1);
    if (j + 2 < X) sqr_row_chain<X, 0>(ue, a, j, j + 2);
  }
  // U = UE + 2^32 UO (< 2^(32 (2X - 1))): no carry out of the top word
  u[0] = ue[0];
  u[1] = add_cc(ue[1], uo[0]);
#pragma unroll
  for (int w = 2; w < 2 * X - 1; w++) u[w] = addc_cc(ue[w], uo[w - 1]);
  u[2 * X - 1] = addc_end(ue[2 * X - 1], uo[2 * X - 2]);
  // v = 2 U + D
#pragma unroll
  for (int i = 0; i < X; i++) {
    const uint32_t d0 = __funnelshift_l(i == 0 ? 0u : u[2 * i - 1], u[2 * i], 1);
    const uint32_t d1 = __funnelshift_l(u[2 * i], u[2 * i + 1], 1);
    if (i == 0)
      asm volatile("mad.lo.cc.u32 %0, %1, %1, %2;" : "=r"(v[0]) : "r"(a[0]), "r"(d0));
    else
      asm volatile("madc.lo.cc.u32 %0, %1, %1, %2;" : "=r"(v[2 * i]) : "r"(a[i]), "r"(d0));
    if (i == X - 1)
      asm volatile("madc.hi.u32 %0, %1, %1, %2;" : "=r"(v[2 * i + 1]) : "r"(a[i]), "r"(d1));
    else
      asm volatile("madc.hi.cc.u32 %0, %1, %1, %2;" : "=r"(v[2 * i + 1]) : "r"(a[i]), "r"(d1));
  }
}

// FLB_TC_TRISQ == 2: a^2 = L^2 + 2 L H 2^(32 X/2) + H^2 2^(32 X) with a = L + H 2^(32 X/2): the two
// half-size triangular squares are independent chains written to disjoint halves of v, the L H
// block (X/2 rows of local_row, two chains per row) is doubled into words [X/2, 3X/2) with the carry
// rippled to the top; the same X (X + 1) / 2 limb products as sqr_local<X>, more independent chains
template <int X>
__device__ __forceinline__ void sqr_local_split(uint32_t (&v)[2 * X], const uint32_t (&a)[X]) {
  constexpr int H = X / 2;
  uint32_t lo[H], hi[H], sl[X], sh[X], m[X];
#pragma unroll
  for (int j = 0; j < H; j++) { lo[j] = a[j]; hi[j] = a[H + j]; }
  sqr_local<H>(sl, lo);
  sqr_local<H>(sh, hi);
  {
    uint32_t E[H + 1], O[H + 1], pend = 0;
#pragma unroll
    for (int t = 0; t <= H; t++) { E[t] = 0; O[t] = 0; }
#pragma unroll
    for (int j = 0; j < H; j++) m[j] = local_row<H>(E, O, pend, lo, hi[j]);
    asm volatile("add.cc.u32 %0, %1, %2;" : "=r"(m[H]) : "r"(E[0]), "r"(pend));
#pragma unroll
    for (int t = 1; t < H; t++) asm volatile("addc.cc.u32 %0, %1, %2;" : "=r"(m[H + t]) : "r"(E[t]), "r"(O[t - 1]));
  }
#pragma unroll
  for (int i = 0; i < X; i++) { v[i] = sl[i]; v[X + i] = sh[i]; }
  uint32_t prev = 0;
#pragma unroll
  for (int t = 0; t < X; t++) {
    const uint32_t d = __funnelshift_l(prev, m[t], 1);
    prev = m[t];
    if (t == 0)
      asm volatile("add.cc.u32 %0, %0, %1;" : "+r"(v[H]) : "r"(d));
    else
      asm volatile("addc.cc.u32 %0, %0, %1;" : "+r"(v[H + t]) : "r"(d));
  }
  const uint32_t top = prev >> 31;
  asm volatile("addc.cc.u32 %0, %0, %1;" : "+r"(v[H + X]) : "r"(top));
#pragma unroll
  for (int w = H + X + 1; w < 2 * X - 1; w++) asm volatile("addc.cc.u32 %0, %0, 0;" : "+r"(v[w]));
  asm volatile("addc.u32 %0, %0, 0;" : "+r"(v[2 * X - 1]));
}

template <int X, int SQ = FLB_TC_TRISQ>
__device__ __forceinline__ void sqr_diag(uint32_t (&v)[2 * X], const uint32_t (&a)[X]) {
  if constexpr (SQ == 2) sqr_local_split<X>(v, a); else sqr_local<X>(v, a);
}

// address of t's word w (w % 4 == 0) for element elem: words [0, S) in the sA row, [S, 2S) in the work
// row.  With w % 4 == 0 the core-matrix offset of word w is cm_off(elem, 0) + 32 w (16-byte K chunks
// 128 bytes apart), so a runtime w costs a shift-add and a select, the element bases are shared.
template <int S>
__device__ __forceinline__ uint4* t_chunk(uint8_t* sA, uint32_t* sW, int elem, int w) {
  using C = Cfg<S>;
  if constexpr (S >= 128) {
    uint8_t* const a = sA + cm_off((uint32_t)elem, 0u, C::KCH) + 32u * (uint32_t)w;
    uint8_t* const b = reinterpret_cast<uint8_t*>(sW + elem * C::WROW + wpad<S>(w - S));
    return reinterpret_cast<uint4*>(w < S ? a : b);
  } else {  // (measured: the select-free form below issues fewer instructions at S <= 64)
    return w < S ? reinterpret_cast<uint4*>(sA + cm_off(elem, 4u * w, C::KCH))
                 : reinterpret_cast<uint4*>(sW + elem * C::WROW + wpad<S>(w - S));
  }
}

// address of t's word w (any w) for element elem (8-byte aligned for even w)
template <int S>
__device__ __forceinline__ uint32_t* t_word(uint8_t* sA, uint32_t* sW, int elem, int w) {
  using C = Cfg<S>;
  return w < S ? reinterpret_cast<uint32_t*>(sA + cm_off((uint32_t)elem, 4u * (uint32_t)w, C::KCH))
               : sW + elem * C::WROW + wpad<S>(w - S);
}

// t[w0 .. w0 + NW) += 2 v (mod 2^(32 NW)); returns the carry out of the region (0..2).  One carry
// chain (add.cc / addc.cc, one IADD3.X per word) across the chunks; the doubling is a funnel shift.
// HEAD = w0 % 4 (0 or 2): a region that starts or ends half-way into a 16-byte chunk (X = 12 limbs per
// lane at S = 96) takes a uint2 at that end.
template <int S, int NW, bool DBL = true, int HEAD = 0>
__device__ __forceinline__ uint32_t t_add_dbl(uint8_t* sA, uint32_t* sW, int elem, int w0, const uint32_t (&v)[NW]) {
  static_assert((HEAD == 0 || HEAD == 2) && (NW - HEAD) % 2 == 0, "whole 8-byte pieces");
  constexpr int NC = (NW - HEAD) / 4, TAIL = (NW - HEAD) % 4;
  uint32_t prev = 0, cy;
  auto add = [&](uint32_t m, int i) {
    const uint32_t x = v[i];
    const uint32_t d = DBL ? __funnelshift_l(prev, x, 1) : x;  // (x << 1) | (prev >> 31)
    prev = x;
    uint32_t r;
    if (i == 0)
      asm volatile("add.cc.u32 %0, %1, %2;" : "=r"(r) : "r"(m), "r"(d));
    else
      asm volatile("addc.cc.u32 %0, %1, %2;" : "=r"(r) : "r"(m), "r"(d));
    return r;
  };
  if constexpr (HEAD == 2) {
    uint2* p = reinterpret_cast<uint2*>(t_word<S>(sA, sW, elem, w0));
    const uint2 m = *p;
    const uint32_t r0 = add(m.x, 0), r1 = add(m.y, 1);
    *p = make_uint2(r0, r1);
  }
#pragma unroll
  for (int c = 0; c < NC; c++) {
    uint4* p = t_chunk<S>(sA, sW, elem, w0 + HEAD + 4 * c);
    const uint4 m = *p;
    const uint32_t r0 = add(m.x, HEAD + 4 * c), r1 = add(m.y, HEAD + 4 * c + 1);
    const uint32_t r2 = add(m.z, HEAD + 4 * c + 2), r3 = add(m.w, HEAD + 4 * c + 3);
    *p = make_uint4(r0, r1, r2, r3);
  }
  if constexpr (TAIL == 2) {
    uint2* p = reinterpret_cast<uint2*>(t_word<S>(sA, sW, elem, w0 + NW - 2));
    const uint2 m = *p;
    const uint32_t r0 = add(m.x, NW - 2), r1 = add(m.y, NW - 1);
    *p = make_uint2(r0, r1);
  }
  asm volatile("addc.u32 %0, 0, 0;" : "=r"(cy));
  return cy + (DBL ? prev >> 31 : 0u);
}

// q[j0 .. N) += the small addends add(j) (each < 2^32, nonzero at a few positions) with one carry
// chain; returns the carry out of q[N - 1]
template <int N, int J0, typename F>
__device__ __forceinline__ uint32_t add_sparse_chain(uint32_t (&q)[N], F add) {
  uint32_t cy;
#pragma unroll
  for (int j = J0; j < N; j++) {
    if (j == J0)
      asm volatile("add.cc.u32 %0, %0, %1;" : "+r"(q[j]) : "r"(add(j)));
    else
      asm volatile("addc.cc.u32 %0, %0, %1;" : "+r"(q[j]) : "r"(add(j)));
  }
  asm volatile("addc.u32 %0, 0, 0;" : "=r"(cy));
  return cy;
}

template <int S, int SQ = FLB_TC_TRISQ>
__device__ __forceinline__ void tc_square_product(const uint32_t (&a)[Cfg<S>::X], int elem, uint8_t* sA,
                                                  uint32_t* sW) {
  constexpr int X = Cfg<S>::X, H = X / 2;
  const int k = threadIdx.x % kT;
  uint32_t cF = 0, cH = 0;
  {
    // diagonal block: t[2Xk, 2Xk + 2X) = a_k^2 (the four tile t exactly)
    uint32_t v[2 * X];
    sqr_diag<X, SQ>(v, a);
    __syncwarp();  // every lane of the group has read its a (it may come from the work row)
#pragma unroll
    for (int c = 0; c < X / 2; c++)
      *t_chunk<S>(sA, sW, elem, 2 * X * k + 4 * c) = make_uint4(v[4 * c], v[4 * c + 1], v[4 * c + 2], v[4 * c + 3]);
  }
  {
    // full off-diagonal block a_k a_l, l = k + 1 mod 4, doubled, at words X (k + l) (lane 3: X 3)
    uint32_t v[2 * X];
    const int l = (k + 1) & (kT - 1);
    blk_prod<X, X>(v, a, a, l, false);
    const int w0 = X * (k < kT - 1 ? 2 * k + 1 : kT - 1);
    __syncwarp();
    if (k < kT - 1) cF = t_add_dbl<S, 2 * X>(sA, sW, elem, w0, v);  // [X, 3X), [3X, 5X), [5X, 7X)
    __syncwarp();
    if (k == kT - 1) cF = t_add_dbl<S, 2 * X>(sA, sW, elem, w0, v);  // [3X, 5X)
  }
  {
    // half block: a_(k&1) x a_((k&1)+2)[H (k>>1), + H), doubled, at words 2X (k&1) + 2X + H (k>>1)
    uint32_t M[X], v[X + H];
    const int i = k & 1, hh = k >> 1;
#pragma unroll
    for (int j = 0; j < X; j++) M[j] = __shfl_sync(FULL, a[j], i, kT);
    // rows [0, H) of a_(i+2) come from lane i + 2 (read by lane i); lane i + 2 itself (hh = 1) takes
    // its own rows [H, X)
    blk_prod<X, H>(v, M, a, i + 2, hh == 1);
    const int w0 = 2 * X * i + 2 * X + H * hh;
    __syncwarp();
    if (hh == 0) cH = t_add_dbl<S, X + H>(sA, sW, elem, w0, v);  // [2X, 3.5X), [4X, 5.5X)
    __syncwarp();
    if (hh == 1) cH = t_add_dbl<S, X + H>(sA, sW, elem, w0, v);  // [2.5X, 4X), [4.5X, 6X)
    __syncwarp();
  }
  // fold the carries into lane k's quarter [2Xk, 2Xk + 2X): at relative offsets 0, X, 1.5X
  //   q1: X <- cF(0), 1.5X <- cH(0);  q2: 0 <- cH(2), X <- cF(1) + cF(3), 1.5X <- cH(1);
  //   q3: 0 <- cH(3), X <- cF(2)
  const uint32_t f0 = __shfl_sync(FULL, cF, 0, kT), f1 = __shfl_sync(FULL, cF, 1, kT);
  const uint32_t f2 = __shfl_sync(FULL, cF, 2, kT), f3 = __shfl_sync(FULL, cF, 3, kT);
  const uint32_t h0 = __shfl_sync(FULL, cH, 0, kT), h1 = __shfl_sync(FULL, cH, 1, kT);
  const uint32_t at0 = k >= 2 ? cH : 0u;
  const uint32_t atX = k == 1 ? f0 : k == 2 ? f1 + f3 : k == 3 ? f2 : 0u;
  const uint32_t atH = k == 1 ? h0 : k == 2 ? h1 : 0u;
  uint32_t q[2 * X];
#pragma unroll
  for (int c = 0; c < X / 2; c++) {
    const uint4 u = *t_chunk<S>(sA, sW, elem, 2 * X * k + 4 * c);
    q[4 * c] = u.x; q[4 * c + 1] = u.y; q[4 * c + 2] = u.z; q[4 * c + 3] = u.w;
  }
  const uint32_t cy = add_sparse_chain<2 * X, 0>(q, [&](int j) { return j == 0 ? at0 : j == X ? atX : j == X + H ? atH : 0u; });
  const uint32_t c = group_carry<kT>(cy != 0, all_ones<2 * X>(q), 0);
  add_word_propagate<2 * X>(q, c & 1u);
#pragma unroll
  for (int cc = 0; cc < X / 2; cc++)
    *t_chunk<S>(sA, sW, elem, 2 * X * k + 4 * cc) = make_uint4(q[4 * cc], q[4 * cc + 1], q[4 * cc + 2], q[4 * cc + 3]);
}

// Block squaring for eight lanes per element (S = 128, X = 16), the T = 4 scheme widened: lane k
// computes its diagonal square a_k^2 (stored to its eighth t[2Xk, 2Xk + 2X)), the full cross blocks
// a_k a_((k+d) mod 8) for d = 1, 2, 3 and half of the d = 4 block (row half k / 4 of a_(k%4) a_(k%4+4)),
// each doubled and added in place at word X (k + l), in two disjoint-range phases per round (lanes
// whose block does not wrap, then the ones that do; the two row halves of the d = 4 blocks).  Per
// lane X (X+1)/2 + 3 X^2 + X^2/2 = 1032 limb products, S (S + 1) / 2 over the group.  The carry-out
// (0..2) of every in-place addition lands at the word just past its range; each lane gathers, by
// shuffles, the carries landing in its eighth and folds them in with one group pass and a ballot
// carry-lookahead.
template <int S, int SQ>
__device__ __forceinline__ void tc_square_product_w(const uint32_t (&a)[Cfg<S>::X], int elem, uint8_t* sA,
                                                    uint32_t* sW) {
  constexpr int X = Cfg<S>::X, T = Cfg<S>::T, H = X / 2, HT = T / 2;
  static_assert(T == 8, "eight lanes per element");
  const int k = threadIdx.x % T;
  {
    uint32_t v[2 * X];
    sqr_diag<X, SQ>(v, a);
    __syncwarp();  // every lane of the group has read its a (it may come from the work row)
#pragma unroll
    for (int c = 0; c < X / 2; c++)
      *t_chunk<S>(sA, sW, elem, 2 * X * k + 4 * c) = make_uint4(v[4 * c], v[4 * c + 1], v[4 * c + 2], v[4 * c + 3]);
  }
  uint32_t cw[HT];  // carry-out of each round's in-place addition
#pragma unroll
  for (int d = 1; d < HT; d++) {
    uint32_t v[2 * X];
    const bool wrap = k + d >= T;
    const int w0 = X * (wrap ? 2 * k + d - T : 2 * k + d);
    uint32_t c = 0;
    blk_prod<X, X, T>(v, a, a, (k + d) & (T - 1), false);
    __syncwarp();
    if (!wrap) c = t_add_dbl<S, 2 * X>(sA, sW, elem, w0, v);
    __syncwarp();
    if (wrap) c = t_add_dbl<S, 2 * X>(sA, sW, elem, w0, v);
    cw[d - 1] = c;
  }
  {
    uint32_t M[X], v[X + H];
    const int i = k & (HT - 1), hh = k / HT;
#pragma unroll
    for (int j = 0; j < X; j++) M[j] = __shfl_sync(FULL, a[j], i, T);
    // rows [0, H) of a_(i+4) come from lane i + 4 (read by lane i); lane i + 4 takes its own rows [H, X)
    blk_prod<X, H, T>(v, M, a, i + HT, hh == 1);
    const int w0 = X * (2 * i + HT) + H * hh;
    uint32_t c = 0;
    __syncwarp();
    if (hh == 0) c = t_add_dbl<S, X + H>(sA, sW, elem, w0, v);
    __syncwarp();
    if (hh == 1) c = t_add_dbl<S, X + H, true, H % 4>(sA, sW, elem, w0, v);  // (X = 12: w0 = 2 mod 4)
    __syncwarp();
    cw[HT - 1] = c;
  }
  // the carries landing in this lane's eighth, at offsets 0, H, X, X + H (a carry past word 2S is 0:
  // t = a^2 < 2^(64 S)).  Round d's carry from source lane j lands at word X (2j + d + 2) (no wrap)
  // or X (2j + d - T + 2) (wrap), the half round's at X (2i + T/2 + 1) + H (hh + 1): so lane k takes
  // round d's carry from lanes k - 1 - d/2 and k - (d - 7)/2 (d odd, at offset X) or k - (d - 6)/2
  // (d even, at offset 0), and the half round's from lane k - 2 (hh = 0, at X + H) and lane k + 1
  // (hh = 1, at 0) — the table enumerated and checked against the positions in DESIGN.md §6.
  uint32_t at[4] = {0, 0, 0, 0};
#pragma unroll
  for (int d = 1; d < HT; d++) {
    const int o = (d & 1) ? 2 : 0;
    const int j1 = k - 1 - d / 2;
    const int j2 = (d & 1) ? k - (d - 7) / 2 : k - (d - 6) / 2;
    const uint32_t c1 = __shfl_sync(FULL, cw[d - 1], j1 & (T - 1), T);
    const uint32_t c2 = __shfl_sync(FULL, cw[d - 1], j2 & (T - 1), T);
    if (j1 >= 0 && j1 + d < T) at[o] += c1;
    if (j2 >= T - d && j2 < T) at[o] += c2;
  }
  {
    const uint32_t c1 = __shfl_sync(FULL, cw[HT - 1], (k - 2) & (T - 1), T);  // hh = 0, i = k - 2
    const uint32_t c2 = __shfl_sync(FULL, cw[HT - 1], (k + 1) & (T - 1), T);  // hh = 1, i = k - 3
    if (k >= 2 && k - 2 < HT) at[3] += c1;
    if (k >= 3 && k - 3 < HT) at[0] += c2;
  }
  uint32_t q[2 * X];
#pragma unroll
  for (int c = 0; c < X / 2; c++) {
    const uint4 u = *t_chunk<S>(sA, sW, elem, 2 * X * k + 4 * c);
    q[4 * c] = u.x; q[4 * c + 1] = u.y; q[4 * c + 2] = u.z; q[4 * c + 3] = u.w;
  }
  const uint32_t cy = add_sparse_chain<2 * X, 0>(q, [&](int j) {
    return j == 0 ? at[0] : j == H ? at[1] : j == X ? at[2] : j == X + H ? at[3] : 0u;
  });
  const uint32_t cc = group_carry<T>(cy != 0, all_ones<2 * X>(q), 0);
  add_word_propagate<2 * X>(q, cc & 1u);
#pragma unroll
  for (int c = 0; c < X / 2; c++)
    *t_chunk<S>(sA, sW, elem, 2 * X * k + 4 * c) = make_uint4(q[4 * c], q[4 * c + 1], q[4 * c + 2], q[4 * c + 3]);
}

// Block squaring for two lanes per element (S = 32, X = 16): lane k computes a_k^2 (X x X, stored to
// t[2Xk, 2Xk + 2X)) and half of the cross block, a_0 a_1[H k, + H) (X x H, doubled, added at words
// X + H k), 384 instead of 512 limb products per lane.  The two cross pieces overlap, so they are
// added in two phases; both carries land in lane 1's half and are folded in by lane 1.
template <int S, int SQ = FLB_TC_TRISQ>
__device__ __forceinline__ void tc_square_product_t2(const uint32_t (&a)[Cfg<S>::X], int elem, uint8_t* sA,
                                                     uint32_t* sW) {
  constexpr int X = Cfg<S>::X, H = X / 2;
  const int k = threadIdx.x % 2;
  {
    uint32_t v[2 * X];
    sqr_diag<X, SQ>(v, a);
    __syncwarp();  // both lanes have read a (it may come from the work row)
#pragma unroll
    for (int c = 0; c < X / 2; c++)
      *t_chunk<S>(sA, sW, elem, 2 * X * k + 4 * c) = make_uint4(v[4 * c], v[4 * c + 1], v[4 * c + 2], v[4 * c + 3]);
  }
  uint32_t cx = 0;
  {
    uint32_t M[X], v[X + H];
#pragma unroll
    for (int j = 0; j < X; j++) M[j] = __shfl_sync(FULL, a[j], 0, 2);
    // rows [0, H) of a_1 come from lane 1 (read by lane 0); lane 1 takes its own rows [H, X)
    blk_prod<X, H, 2>(v, M, a, 1, k == 1);
    __syncwarp();
    if (k == 0) cx = t_add_dbl<S, X + H>(sA, sW, elem, X, v);      // [X, 2X + H): carry at 2X + H
    __syncwarp();
    if (k == 1) cx = t_add_dbl<S, X + H>(sA, sW, elem, X + H, v);  // [X + H, 3X): carry at 3X
    __syncwarp();
  }
  const uint32_t c0 = __shfl_sync(FULL, cx, 0, 2);
  if (k == 1) {
    // lane 1's half t[2X, 4X): + c0 at relative H, + cx at relative X (no carry leaves t)
    uint32_t q[2 * X];
#pragma unroll
    for (int c = 0; c < X / 2; c++) {
      const uint4 u = *t_chunk<S>(sA, sW, elem, 2 * X + 4 * c);
      q[4 * c] = u.x; q[4 * c + 1] = u.y; q[4 * c + 2] = u.z; q[4 * c + 3] = u.w;
    }
    add_sparse_chain<2 * X, H>(q, [&](int j) { return j == H ? c0 : j == X ? cx : 0u; });  // (no carry leaves t)
#pragma unroll
    for (int c = H / 4; c < X / 2; c++)
      *t_chunk<S>(sA, sW, elem, 2 * X + 4 * c) = make_uint4(q[4 * c], q[4 * c + 1], q[4 * c + 2], q[4 * c + 3]);
  }
  __syncwarp();
}


// The product phase of tc_mont: t = a b (2S words) for the 128 elements of the tile, t_lo into the
// elements' sA rows (the MMA A operand), t_hi into their work rows.  Groups of T lanes per element
// (X = 16 limbs each), NP passes of EP elements.  CTA-collective (no trailing barrier).
template <int S, int SQ = FLB_TC_TRISQ>
__device__ __forceinline__ void tc_product(const Src& sa, const Src& sb, bool sq, uint8_t* sA, uint32_t* sW,
                                           int np = Cfg<S>::NP) {
  using C = Cfg<S>;
  constexpr int X = C::X, KCH = C::KCH;
  constexpr int T = C::T;
  const int tid = threadIdx.x, k = tid % T;
  // ---- P: t = a b, np passes of EP elements (S = 64: two passes of 64; S = 32: one of 128)
#pragma unroll 1
  for (int h = 0; h < np; h++) {
    const int elem = prod_elem<S>(h);
    uint32_t a[X], b[X];
    src_load<S>(a, sa, elem, sW);
    if constexpr (T == 2) {
      if (sq) {
        tc_square_product_t2<S, SQ>(a, elem, sA, sW);
        continue;
      }
    } else if constexpr (T == 4) {
      if (sq) {
        tc_square_product<S, SQ>(a, elem, sA, sW);
        continue;
      }
    } else {
      if (sq) {
        tc_square_product_w<S, SQ>(a, elem, sA, sW);
        continue;
      }
    }
    src_load<S>(b, sb, elem, sW);
    // stage b in the element's sA row (natural byte order: word w at chunk w / 4)
    __syncwarp();
#pragma unroll
    for (int v = 0; v < X / 4; v++)
      *reinterpret_cast<uint4*>(sA + cm_off(elem, 16u * (k * X / 4 + v), KCH)) =
          make_uint4(b[4 * v], b[4 * v + 1], b[4 * v + 2], b[4 * v + 3]);
    __syncwarp();
    uint32_t E[X + 1], O[X + 1], pend = 0, lo[X], hi[X];
    const uint32_t dummy[X] = {};
#pragma unroll
    for (int t = 0; t <= X; t++) { E[t] = 0; O[t] = 0; }
#pragma unroll
    for (int t = 0; t < X; t++) lo[t] = 0;
#pragma unroll 1
    for (int kk = 0; kk < T; kk++) {
#pragma unroll
      for (int j4 = 0; j4 < X; j4 += 4) {
        const uint4 bq = *reinterpret_cast<const uint4*>(sA + cm_off(elem, 4u * (kk * X + j4), KCH));
        const uint32_t bw[4] = {bq.x, bq.y, bq.z, bq.w};
#pragma unroll
        for (int u = 0; u < 4; u++) {
          const uint32_t o = cios_step<X, T, false>(E, O, pend, a, bw[u], dummy, 0u);
          if (k == kk) lo[j4 + u] = o;
        }
      }
    }
    collapse<X, T>(hi, E, O, pend);
    __syncwarp();
#pragma unroll
    for (int v = 0; v < X / 4; v++) {
      *reinterpret_cast<uint4*>(sA + cm_off(elem, 16u * (k * X / 4 + v), KCH)) =
          make_uint4(lo[4 * v], lo[4 * v + 1], lo[4 * v + 2], lo[4 * v + 3]);
      *reinterpret_cast<uint4*>(sW + elem * C::WROW + wpad<S>(k * X + 4 * v)) =
          make_uint4(hi[4 * v], hi[4 * v + 1], hi[4 * v + 2], hi[4 * v + 3]);
    }
  }
}

// Montgomery product over the tile: for every element, a b R^-1 mod N (canonical) into its work
// row.  sq: b = a.  `phase` tracks the mbarrier parity (two completions per call).  CTA-collective.
// LDP: the normalisation double-buffers its TMEM loads (chunk c + 1 in flight while chunk c is
// normalised) — measured faster in k_tc_exp_dag (245.4 -> 242.1 ms), slower in k_tc_exp.
template <int S, int SQ = FLB_TC_TRISQ, bool LDP = false>
__device__ __forceinline__ void tc_mont(const Src& sa, const Src& sb, bool sq, const Smem& sm,
                                        const uint32_t* __restrict__ Nmod, uint32_t& phase) {
  using C = Cfg<S>;
  constexpr int X = C::X, KCH = C::KCH, KB = C::KB, QW = C::QW, QC = C::QC;
  const int tid = threadIdx.x, warp = tid >> 5;
  uint8_t* sA = sm.base + C::OFF_A;
  uint32_t* sW = reinterpret_cast<uint32_t*>(sm.base + C::OFF_W);
#if FLB_TC_PROF
  long long t_ = clock64();
#endif
  tc_product<S, SQ>(sa, sb, sq, sA, sW, sm.np);
  fence_async_smem();
  tc_before_sync();
  __syncthreads();
  TC_MARK(0);
  // ---- M1: q columns [0, KB)
  if (tid == 0) {
    tc_after_sync();
    mma_toeplitz_lo<KB>(sm.tmem, smem_u32(sA), smem_u32(sm.base + C::OFF_E1));
    mma_commit(sm.mbar);
  }
  // normalisation: TMEM lane quadrant L = warp % 4 (elements 32L ..), column half g = warp / 4
  const int L = warp & 3, g = warp >> 2, i = 32 * L + (tid & 31);
  const bool nw = true;  // every warp normalises: column group g of elements [32 L, 32 L + 32)
  const uint32_t lane_base = sm.tmem + ((uint32_t)(32 * L) << 16);
  uint32_t* row = sW + i * C::WROW;
  // carry exchange per (element, column group): x = carry (< 2^21) | all-ones flag << 29 | borrow,
  // zero flags << 30, y = the group's word 0
  uint2* xch = reinterpret_cast<uint2*>(sm.base + C::OFF_X) + i * C::NG;
  constexpr int NG = C::NG;
  uint2 ttop = make_uint2(0, 0);
  if (g == 0) ttop = *reinterpret_cast<const uint2*>(sA + cm_off(i, KB - 8, KCH));  // t_lo bytes KB-8 ..
  mbar_wait(sm.mbar, phase);
  phase ^= 1u;
  tc_after_sync();
  TC_MARK(1);
  uint32_t v[QW];
  auto add_in = [&](uint64_t cin) {
    v[0] = add_cc(v[0], (uint32_t)cin);
    v[1] = addc_cc(v[1], (uint32_t)(cin >> 32));
#pragma unroll
    for (int w = 2; w < QW; w++) v[w] = addc_cc(v[w], 0u);
  };
  auto publish = [&](uint64_t carry) {
    uint32_t ao = 0xffffffffu;
#pragma unroll
    for (int w = 1; w < QW; w++) ao &= v[w];
    xch[g] = make_uint2((uint32_t)carry | (ao == 0xffffffffu ? 1u << 29 : 0u), v[0]);
  };
  // carry into half 1 (= out of half 0), and out of half 1
  auto carry_out = [&](int h, uint64_t cin) {
    const uint2 x = xch[h];
    const uint64_t ov = ((x.x >> 29) & 1u) != 0u && (((uint64_t)x.y + cin) >> 32) != 0 ? 1u : 0u;
    return (uint64_t)(x.x & 0x1fffffffu) + ov;
  };
  // carry into column group gg (the prefix over the groups below it)
  auto carry_into = [&](int gg) {
    uint64_t c = 0;
#pragma unroll
    for (int h = 0; h < NG - 1; h++)
      if (h < gg) c = carry_out(h, c);
    return c;
  };
  // ---- N1: q = D1 mod R
  if (nw) {
    NormState ns;
    if constexpr (LDP) {
      // the TMEM load of chunk c + 1 is in flight while chunk c is normalised (two 32-column buffers)
      uint32_t ca[32], cb[32];
      tmem_ld32(lane_base + (uint32_t)(g * QC), ca);
      tmem_wait();
#pragma unroll
      for (int c0 = 0; c0 < QC; c0 += 32) {
        uint32_t(&cur)[32] = ((c0 / 32) & 1) ? cb : ca;
        uint32_t(&nxt)[32] = ((c0 / 32) & 1) ? ca : cb;
        if (c0 + 32 < QC) tmem_ld32(lane_base + (uint32_t)(g * QC + c0 + 32), nxt);
        norm8_chain<false>(cur, nullptr, v + c0 / 4, ns, c0 == 0);
        if (c0 + 32 < QC) tmem_wait();
      }
    } else {
#pragma unroll
      for (int c0 = 0; c0 < QC; c0 += 32) {
        uint32_t cv[32];
        tmem_ld32(lane_base + (uint32_t)(g * QC + c0), cv);
        tmem_wait();
        norm8_chain<false>(cv, nullptr, v + c0 / 4, ns, c0 == 0);
      }
    }
    publish(ns.carry_out_end());
  }
  pair_sync<S>();  // carries published (D1 drained before M2: the CTA barrier below)
  if (nw) {
    if (g > 0) add_in(carry_into(g));
#pragma unroll
    for (int c = 0; c < QW / 4; c++)
      *reinterpret_cast<uint4*>(sA + cm_off(i, g * QC + 16 * c, KCH)) =
          make_uint4(v[4 * c], v[4 * c + 1], v[4 * c + 2], v[4 * c + 3]);
  }
  fence_async_smem();
  tc_before_sync();
  __syncthreads();
  // ---- M2: q N columns [KB-8, 2KB-8) into D2 = TMEM [0, KB)
  if (tid == 0) {
    tc_after_sync();
    mma_toeplitz_hi<KB>(sm.tmem, smem_u32(sA), smem_u32(sm.base + C::OFF_E2));
    mma_commit(sm.mbar);
  }
  TC_MARK(2);
  mbar_wait(sm.mbar, phase);
  phase ^= 1u;
  tc_after_sync();
  TC_MARK(3);
  // ---- F: u = t_hi + high(q N) + c'.  t_lo + (q N mod R) = c' R exactly; with W = the 8 byte
  // columns below KB of t + q N (as an integer over those columns) and Z the rest
  // (< 2^(8(KB-8)+26)), c' R = W 2^(8(KB-8)) + Z, so c' = ceil(W / 2^64).  Half 0 starts with c'.
  if (nw) {
    uint64_t carry = 0;
    if (g == 0) {
      uint32_t bc[8];
      tmem_ld8(lane_base, bc);
      tmem_wait();
      // W as two words (the funnel-shift form of norm8_chain, on the ALU pipe)
      const uint64_t s0 = (uint64_t)bc[0] + (bc[1] << 8) + (bc[2] << 16) + (uint64_t)(bc[3] << 24) + ttop.x;
      const uint64_t s1 = (s0 >> 32) + bc[4] + __funnelshift_l(bc[1], bc[5], 8) + __funnelshift_l(bc[2], bc[6], 16) +
                          (uint64_t)__funnelshift_l(bc[3], bc[7], 24) + ttop.y;
      const uint64_t top = (s1 >> 32) + (bc[5] >> 24) + (bc[6] >> 16) + (bc[7] >> 8);
      carry = top + ((((uint32_t)s0) | ((uint32_t)s1)) != 0u ? 1u : 0u);
    }
    NormState ns;
    ns.hprev = (uint32_t)carry;  // < 2^20
    // this group's columns KB + g QC + c, i.e. D2 columns 8 + g QC + c; the last group's last 8
    // columns (2KB-8 .. 2KB-1) are outside D2: the 7 top columns of q N from its top 8 bytes and N's
    uint32_t top[8] = {0, 0, 0, 0, 0, 0, 0, 0};
    if (g == NG - 1) {
      const uint2 qt2 = *reinterpret_cast<const uint2*>(sA + cm_off(i, KB - 8, KCH));
      const uint2 nt2 = __ldg(reinterpret_cast<const uint2*>(Nmod + S - 2));
      uint32_t qt[8], nt[8];
#pragma unroll
      for (int b = 0; b < 4; b++) {
        qt[b] = (qt2.x >> (8 * b)) & 0xffu; qt[4 + b] = (qt2.y >> (8 * b)) & 0xffu;
        nt[b] = (nt2.x >> (8 * b)) & 0xffu; nt[4 + b] = (nt2.y >> (8 * b)) & 0xffu;
      }
#pragma unroll
      for (int j = 0; j < 7; j++) {
        uint32_t acc = 0;
#pragma unroll
        for (int a2 = j + 1; a2 < 8; a2++) acc += qt[a2] * nt[j - a2 + 8];
        top[j] = acc;
      }
    }
    if constexpr (LDP) {
      // as N1: chunk c + 1's TMEM loads overlap chunk c's normalisation
      auto load_chunk = [&](int c0, uint32_t(&cv)[32], uint32_t(&t8)[8]) {
        const uint32_t col = 8u + (uint32_t)(g * QC + c0);
        if (c0 + 32 < QC) {
          tmem_ld32(lane_base + col, cv);
        } else {  // D2 columns col + 24 .. col + 31 exist for all but the last group (its top columns)
          tmem_ld16(lane_base + col, cv);
          tmem_ld8(lane_base + col + 16u, cv + 16);
          tmem_ld8(lane_base + (g < NG - 1 ? col + 24u : 0u), t8);  // uniform per warp; unused for the last
        }
      };
      auto fix_last = [&](int c0, uint32_t(&cv)[32], const uint32_t(&t8)[8]) {
        if (c0 + 32 >= QC) {
#pragma unroll
          for (int j = 0; j < 8; j++) cv[24 + j] = g < NG - 1 ? t8[j] : top[j];
        }
      };
      uint32_t ca[32], cb[32], t8[8];
      load_chunk(0, ca, t8);
      tmem_wait();
      fix_last(0, ca, t8);
#pragma unroll
      for (int c0 = 0; c0 < QC; c0 += 32) {
        uint32_t(&cur)[32] = ((c0 / 32) & 1) ? cb : ca;
        uint32_t(&nxt)[32] = ((c0 / 32) & 1) ? ca : cb;
        if (c0 + 32 < QC) load_chunk(c0 + 32, nxt, t8);
        const uint4 h0 = reinterpret_cast<const uint4*>(row + wpad<S>(g * QW + c0 / 4))[0];  // 8 words, one 32-block
        const uint4 h1 = reinterpret_cast<const uint4*>(row + wpad<S>(g * QW + c0 / 4))[1];
        const uint32_t th[8] = {h0.x, h0.y, h0.z, h0.w, h1.x, h1.y, h1.z, h1.w};
        norm8_chain<true>(cur, th, v + c0 / 4, ns, c0 == 0);
        if (c0 + 32 < QC) {
          tmem_wait();
          fix_last(c0 + 32, nxt, t8);
        }
      }
    } else {
#pragma unroll
      for (int c0 = 0; c0 < QC; c0 += 32) {
        uint32_t cv[32];
        const uint32_t col = 8u + (uint32_t)(g * QC + c0);
        if (c0 + 32 < QC) {
          tmem_ld32(lane_base + col, cv);
        } else {
          // last chunk of the group: D2 columns col .. col+23 always exist; col+24 .. col+31 exist
          // for all but the last group (whose are the top columns)
          tmem_ld16(lane_base + col, cv);
          tmem_ld8(lane_base + col + 16u, cv + 16);
          uint32_t t8[8];
          tmem_ld8(lane_base + (g < NG - 1 ? col + 24u : 0u), t8);  // uniform per warp; unused for the last
          tmem_wait();
#pragma unroll
          for (int j = 0; j < 8; j++) cv[24 + j] = g < NG - 1 ? t8[j] : top[j];
        }
        tmem_wait();
        const uint4 h0 = reinterpret_cast<const uint4*>(row + wpad<S>(g * QW + c0 / 4))[0];  // 8 words, one 32-block
        const uint4 h1 = reinterpret_cast<const uint4*>(row + wpad<S>(g * QW + c0 / 4))[1];
        const uint32_t th[8] = {h0.x, h0.y, h0.z, h0.w, h1.x, h1.y, h1.z, h1.w};
        norm8_chain<true>(cv, th, v + c0 / 4, ns, c0 == 0);
      }
    }
    publish(ns.carry_out_end());
  }
  pair_sync<S>();
  uint64_t ovf = 0;
  uint32_t d[QW];
  if (nw) {
    const uint64_t cg = carry_into(g);
    ovf = carry_out(NG - 1, carry_into(NG - 1));  // bit above S words (u < 2N < 2R)
    if (g > 0) add_in(cg);
    // u - N over this group: local borrow and zero-difference flag
    uint32_t br = 0, nzd = 0;
    uint32_t nn[QW];
#pragma unroll
    for (int c = 0; c < QW / 4; c++) {
      const uint4 nv = __ldg(reinterpret_cast<const uint4*>(Nmod + g * QW + 4 * c));
      nn[4 * c] = nv.x; nn[4 * c + 1] = nv.y; nn[4 * c + 2] = nv.z; nn[4 * c + 3] = nv.w;
    }
    d[0] = sub_cc(v[0], nn[0]);
#pragma unroll
    for (int w = 1; w < QW; w++) d[w] = subc_cc(v[w], nn[w]);
    br = subc_end(0u, 0u) & 1u;
#pragma unroll
    for (int w = 0; w < QW; w++) nzd |= d[w];
    xch[g].x |= (br | (nzd == 0u ? 2u : 0u)) << 30;  // (the pair reads only bits < 30 concurrently)
  }
  pair_sync<S>();
  if (nw) {
    // borrow into each group: b_(h+1) = borrow_h | (zero_h & b_h); bout = the borrow out of the top
    uint32_t bin = 0, bout = 0;
#pragma unroll
    for (int h = 0; h < NG; h++) {
      if (h == g) bin = bout;
      const uint32_t f = xch[h].x >> 30;
      bout = (f & 1u) | ((f >> 1) & bout);
    }
    if (ovf != 0 || bout == 0) {                           // u >= N: take u - N
      v[0] = sub_cc(d[0], bin);
#pragma unroll
      for (int w = 1; w < QW; w++) v[w] = subc_cc(d[w], 0u);
    }
#pragma unroll
    for (int c = 0; c < QW / 4; c++)
      *reinterpret_cast<uint4*>(row + wpad<S>(g * QW + 4 * c)) = make_uint4(v[4 * c], v[4 * c + 1], v[4 * c + 2], v[4 * c + 3]);
  }
  tc_before_sync();
  pair_sync<S>();  // the pair's rows are final (the next product / row op of these elements is the pair's)
  TC_MARK(4);
#if FLB_TC_PROF
  if (threadIdx.x == 0) atomicAdd(&g_tc_prof[(S == 64 ? 8 : 0) + 5], 1ull);
#endif
}

// copy each element's work row (words 0..S-1) to dst + j * stride (elements j < valid; j = unit_index of
// the row when half)
template <int S>
__device__ __forceinline__ void tc_row_store(const Smem& sm, uint32_t* dst, uint32_t stride, uint32_t valid,
                                             bool half = false) {
  using C = Cfg<S>;
  const uint32_t* sW = reinterpret_cast<const uint32_t*>(sm.base + C::OFF_W);
  const int k = threadIdx.x % C::T;
#pragma unroll 1
  for (int h = 0; h < sm.np; h++) {
    const int elem = prod_elem<S>(h);
    const int j = unit_index(elem, half);
    if ((uint32_t)j < valid) {
      const uint4* q = reinterpret_cast<const uint4*>(sW + elem * C::WROW + wpad<S>(k * C::X));
      uint4* o = reinterpret_cast<uint4*>(dst + (size_t)j * stride + k * C::X);
#pragma unroll
      for (int v = 0; v < C::X / 4; v++) o[v] = q[v];
    }
  }
}

// work row <- (row + 1) mod N for every element (row < N)
template <int S>
__device__ __forceinline__ void tc_row_add_one(const Smem& sm, const uint32_t* __restrict__ Nmod) {
  using C = Cfg<S>;
  constexpr int X = C::X;
  uint32_t* sW = reinterpret_cast<uint32_t*>(sm.base + C::OFF_W);
  const int k = threadIdx.x % C::T;
#pragma unroll 1
  for (int h = 0; h < sm.np; h++) {
    const int elem = prod_elem<S>(h);
    uint32_t r[X], nn[X];
    src_load<S>(r, src_row(), elem, sW);
    load_const<X, C::T>(nn, Nmod);
    grp_add_small<X, C::T>(r, 1u);
    grp_cond_sub<X, C::T>(r, nn, 0u);
    uint4* o = reinterpret_cast<uint4*>(sW + elem * C::WROW + wpad<S>(k * X));
#pragma unroll
    for (int v = 0; v < X / 4; v++) o[v] = make_uint4(r[4 * v], r[4 * v + 1], r[4 * v + 2], r[4 * v + 3]);
  }
  pair_sync<S>();
}

// work row <- (row + s) mod N for every element (row, s < N)
template <int S>
__device__ __forceinline__ void tc_row_add(const Smem& sm, const Src& s, const uint32_t* __restrict__ Nmod) {
  using C = Cfg<S>;
  constexpr int X = C::X;
  uint32_t* sW = reinterpret_cast<uint32_t*>(sm.base + C::OFF_W);
  const int k = threadIdx.x % C::T;
#pragma unroll 1
  for (int h = 0; h < sm.np; h++) {
    const int elem = prod_elem<S>(h);
    uint32_t r[X], a[X], nn[X];
    src_load<S>(r, src_row(), elem, sW);
    src_load<S>(a, s, elem, sW);
    load_const<X, C::T>(nn, Nmod);
    const uint32_t cy = grp_add<X, C::T>(r, r, a);
    grp_cond_sub<X, C::T>(r, nn, cy);
    uint4* o = reinterpret_cast<uint4*>(sW + elem * C::WROW + wpad<S>(k * X));
#pragma unroll
    for (int v = 0; v < X / 4; v++) o[v] = make_uint4(r[4 * v], r[4 * v + 1], r[4 * v + 2], r[4 * v + 3]);
  }
  pair_sync<S>();
}

// ----------------------------------------------------------------------------- batched modexp
// One modular exponentiation per element with an exponent shared by the batch (the
// windowed modexp of Alg. 2's Montgomery product), every Montgomery product by tc_mont.  A launch
// serves up to two problems (the two CRT primes); its tiles are numbered problem 0 first, and a
// persistent CTA reloads the Toeplitz operands when it crosses into the other problem.
//   input  x: x_words <= S words per element (x R = mont(x, R^2)), or 2S words split as lo + hi R
//         (x R = mont(lo, R^2) + mont(hi, R^3)), i.e. a 2S-word integer entering the S-word frame
//   output m == null: x^E mod N (canonical);  m != null: (1 + m n) x^E mod N (Eq. 3,
//         g = n + 1, for the key-holder encryption with x = r^Q mod P and E = P)
// The odd-power window table of each element lives in global scratch [entry][elem][S] per CTA
// (entry `table` holds x^2, then the saved power).
struct ExpProblem {
  const uint32_t* N;       // modulus (S words)
  const uint32_t* R2;      // R^2 mod N
  const uint32_t* R3;      // R^3 mod N (two-half input only)
  const uint32_t* E1;      // extended Toeplitz(N') operand, 2KB x 32 bytes (core matrices)
  const uint32_t* E2;      // extended Toeplitz(N) operand, 3KB x 32 bytes
  const uint32_t* sched;   // exponent schedule (at least one op after the first window)
  int sched_len, table;
  const uint32_t* x;       // [count][x_stride]
  uint32_t x_stride, x_words;
  const uint32_t* m;       // [count][m_stride] (m_words limbs) or null
  uint32_t m_stride, m_words;
  const uint32_t* nR;      // n R mod N (with m)
  uint32_t* out;           // [count][S]
  uint64_t count, tiles;
};
struct ExpArgs {
  ExpProblem pb[2];
  int nprob;
  int half_units;          // the incomplete last round as half units (0: another launch fills the tail)
  const uint32_t* one;     // the integer 1 (at least one word)
  uint32_t* scratch;       // gridDim * kTileM * tab_entries * S words
  int tab_entries;         // max table over the problems + 1 (the per-CTA scratch stride)
};

template <int S>
__device__ __forceinline__ void tc_load_operands(uint8_t* smem, const ExpProblem& P) {
  using C = Cfg<S>;
  constexpr int KB = C::KB;
  const uint4* s1 = reinterpret_cast<const uint4*>(P.E1);
  const uint4* s2 = reinterpret_cast<const uint4*>(P.E2);
  uint4* d1 = reinterpret_cast<uint4*>(smem + C::OFF_E1);
  uint4* d2 = reinterpret_cast<uint4*>(smem + C::OFF_E2);
  for (int i = threadIdx.x; i < 2 * KB * 32 / 16; i += C::THREADS) d1[i] = __ldg(s1 + i);
  for (int i = threadIdx.x; i < 3 * KB * 32 / 16; i += C::THREADS) d2[i] = __ldg(s2 + i);
  fence_async_smem();
}

// One tile (128 elements) of problem P: the element powers x^E (or (1 + m n) x^E) into P.out.  `tab`
// is the CTA's window-table scratch ([entry][kTileM][S] words).  The Toeplitz operands of P are in
// shared memory (tc_load_operands).  hf >= 0: half unit hf of the tile (its elements 64 hf .. 64 hf + 63
// on the rows of product pass 0, sm.np = 1).
template <int S, int SQ = FLB_TC_TRISQ, bool LDP = false>
__device__ __forceinline__ void tc_exp_tile(const ExpProblem& P, uint64_t tile, const uint32_t* one, uint32_t* tab,
                                            const Smem& sm, uint32_t& phase, uint32_t x_ld = kLdNC, int hf = -1) {
  const Src row = src_row();
  const int TB = P.table;
  const bool half = hf >= 0;
  auto slot = [&](int ent) { return src_arr(tab + (size_t)ent * kTileM * S, S, S, kTileM, kLdCTA); };
  auto slot_ptr = [&](int ent) { return tab + (size_t)ent * kTileM * S; };
  const uint64_t e0 = tile * kTileM + (half ? (uint64_t)(kTileM / 2) * hf : 0u);
  const uint64_t cap = half ? kTileM / 2 : kTileM;
  // (the second half unit of a last tile with <= 64 elements is empty)
  const uint32_t nvalid = e0 >= P.count ? 0u : (uint32_t)((P.count - e0) < cap ? (P.count - e0) : cap);
  const uint32_t* xb = P.x + e0 * P.x_stride;
  if (P.x_words <= (uint32_t)S) {
    tc_mont<S, SQ, LDP>(src_arr(xb, P.x_stride, P.x_words, nvalid, x_ld, half), src_arr(P.R2, 0, S, kTileM), false, sm,
                   P.N, phase);
  } else {
    tc_mont<S, SQ, LDP>(src_arr(xb, P.x_stride, S, nvalid, x_ld, half), src_arr(P.R2, 0, S, kTileM), false, sm, P.N, phase);
    tc_row_store<S>(sm, slot_ptr(0), S, kTileM);            // lo R
    tc_mont<S, SQ, LDP>(src_arr(xb + S, P.x_stride, P.x_words - S, nvalid, x_ld, half), src_arr(P.R3, 0, S, kTileM), false,
                   sm, P.N, phase);                         // hi R^2
    tc_row_add<S>(sm, slot(0), P.N);
  }
  tc_row_store<S>(sm, slot_ptr(0), S, kTileM);              // x R mod N
  if (TB > 1) {
    tc_mont<S, SQ, LDP>(row, row, true, sm, P.N, phase);             // x^2
    tc_row_store<S>(sm, slot_ptr(TB), S, kTileM);
#pragma unroll 1
    for (int t = 1; t < TB; t++) {
      tc_mont<S, SQ, LDP>(slot(t - 1), slot(TB), false, sm, P.N, phase);
      tc_row_store<S>(sm, slot_ptr(t), S, kTileM);
    }
  }
  const uint32_t op0 = __ldg(P.sched);
  Src cur = slot((int)(op0 >> 16) - 1);
#pragma unroll 1
  for (int o = 1; o < P.sched_len; o++) {
    const uint32_t op = __ldg(P.sched + o);
    const int sq = (int)(op & 0xffffu), idx = (int)(op >> 16) - 1;
#pragma unroll 1
    for (int t = 0; t < sq; t++) {
      tc_mont<S, SQ, LDP>(cur, cur, true, sm, P.N, phase);
      cur = row;
    }
    if (idx >= 0) {
      tc_mont<S, SQ, LDP>(cur, slot(idx), false, sm, P.N, phase);
      cur = row;
    }
  }
  if (P.m) {
    tc_row_store<S>(sm, slot_ptr(TB), S, kTileM);           // x^E R
    tc_mont<S, SQ, LDP>(src_arr(P.m + e0 * P.m_stride, P.m_stride, P.m_words, nvalid, kLdNC, half),
                   src_arr(P.nR, 0, S, kTileM), false, sm, P.N, phase);  // m n
    tc_row_add_one<S>(sm, P.N);                             // 1 + m n mod N
    tc_mont<S, SQ, LDP>(slot(TB), row, false, sm, P.N, phase);       // (1 + m n) x^E
  } else {
    tc_mont<S, SQ, LDP>(row, src_arr(one, 0, 1, kTileM), false, sm, P.N, phase);  // leave the Montgomery domain
  }
  tc_row_store<S>(sm, P.out + e0 * S, S, nvalid, half);
}

// CTA prologue / epilogue shared by the modexp kernels: the MMA-completion mbarrier and COLS TMEM columns
template <int COLS>
__device__ __forceinline__ void tc_cta_init(uint64_t* mbar, uint32_t* tmem_sh) {
  if (threadIdx.x == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" :: "r"(smem_u32(mbar)));
    asm volatile("fence.mbarrier_init.release.cluster;");
  }
  if ((threadIdx.x >> 5) == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" :: "r"(smem_u32(tmem_sh)),
                 "n"(COLS));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  tc_before_sync();
  __syncthreads();
  tc_after_sync();
}
template <int COLS>
__device__ __forceinline__ void tc_cta_fini(uint32_t tmem) {
  tc_before_sync();
  __syncthreads();
  if ((threadIdx.x >> 5) == 0) {
    tc_after_sync();
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" :: "r"(tmem), "n"(COLS));
  }
}

template <int S>
__global__ void __launch_bounds__(Cfg<S>::THREADS, Cfg<S>::CTAS_PER_SM) k_tc_exp(const ExpArgs A) {
  using C = Cfg<S>;
  extern __shared__ __align__(1024) uint8_t smem[];
  __shared__ __align__(8) uint64_t mbar;
  __shared__ uint32_t tmem_sh;
  tc_cta_init<C::TMEM_COLS>(&mbar, &tmem_sh);
  const Smem sm{smem, tmem_sh, &mbar, C::NP};
  const Smem sm_half{smem, tmem_sh, &mbar, 1};
  uint32_t phase = 0;
  const uint64_t tiles_all = A.pb[0].tiles + (A.nprob > 1 ? A.pb[1].tiles : 0);
  // The K tiles of an incomplete last round run as 2K half units of one product pass (≈ 0.6 of a
  // tile's time) when that still fits one round (2K <= grid): a shorter tail.
  const uint64_t rem = tiles_all % gridDim.x;
  const uint64_t K = (A.half_units && C::NP == 2 && 2 * rem <= gridDim.x) ? rem : 0;
  const uint64_t units = tiles_all + K;
  int loaded = -1;
  uint32_t* tab = A.scratch + (size_t)blockIdx.x * kTileM * A.tab_entries * S;
  for (uint64_t u = blockIdx.x; u < units; u += gridDim.x) {
    const bool whole = u < tiles_all - K;
    const uint64_t gt = whole ? u : tiles_all - K + (u - (tiles_all - K)) / 2;
    const int hf = whole ? -1 : (int)((u - (tiles_all - K)) & 1u);
    const int pi = gt < A.pb[0].tiles ? 0 : 1;
    const ExpProblem& P = A.pb[pi];
    if (pi != loaded) {
      __syncthreads();  // the previous problem's MMAs completed (waited on) before the overwrite
      tc_load_operands<S>(smem, P);
      tc_before_sync();
      __syncthreads();
      loaded = pi;
    }
    tc_exp_tile<S, FLB_TC_TRISQ_EXP>(P, pi == 0 ? gt : gt - A.pb[0].tiles, A.one, tab, whole ? sm : sm_half, phase,
                                     kLdNC, hf);
    __syncthreads();  // the work rows are rewritten by the next tile's first product
  }
  tc_cta_fini<C::TMEM_COLS>(tmem_sh);
}

// Key-holder encryption, both stages in one persistent launch (a dependency DAG instead of two
// launches): the work queue holds the stage-1 tiles of A1 (y = r^Q mod P in the S1-word frame, both
// primes) and then the stage-2 tiles of A2 ((1 + m n) y^P mod P^2 in the S2-word frame), taken
// dynamically from a global counter.  Stage-2 tile j reads exactly the rows stage-1 tile j wrote
// (same counts, same tile numbering), so it waits for tile j's flag (release / acquire at gpu
// scope).  Every stage-1 tile is dequeued before any stage-2 tile, by a running CTA, so the wait
// always ends.  Compared with two launches, the last partial round of stage 1 no longer idles the
// GPU and the end-of-launch tail is at most one stage-2 tile per CTA slot.
// sync: [0] the tile counter, [1 + j] the flag of stage-1 tile j (zeroed before the launch).
template <int S1, int S2>
__global__ void __launch_bounds__(Cfg<S2>::THREADS, 2) k_tc_exp_dag(const ExpArgs A1, const ExpArgs A2, uint32_t* sync,
                                                           uint64_t tab_stride) {
  constexpr int COLS = Cfg<S1>::TMEM_COLS > Cfg<S2>::TMEM_COLS ? Cfg<S1>::TMEM_COLS : Cfg<S2>::TMEM_COLS;
  extern __shared__ __align__(1024) uint8_t smem[];
  __shared__ __align__(8) uint64_t mbar;
  __shared__ uint32_t tmem_sh, next;
  tc_cta_init<COLS>(&mbar, &tmem_sh);
  const Smem sm1{smem, tmem_sh, &mbar, Cfg<S1>::NP}, sm2{smem, tmem_sh, &mbar, Cfg<S2>::NP};
  const Smem sm2h{smem, tmem_sh, &mbar, 1};
  uint32_t phase = 0;
  const uint64_t T1 = A1.pb[0].tiles + A1.pb[1].tiles, T2 = A2.pb[0].tiles + A2.pb[1].tiles;
  // the last K2 stage-2 tiles (those beyond whole rounds of the grid) run as 2 K2 half units (as in
  // k_tc_exp): the queue holds T1 stage-1 tiles, then T2 - K2 stage-2 tiles, then 2 K2 half units
  const uint64_t rem2 = T2 % gridDim.x;
  const uint64_t K2 = (A2.half_units && Cfg<S2>::NP == 2 && 2 * rem2 <= gridDim.x) ? rem2 : 0;
  const uint64_t U2 = T2 + K2;
  int loaded = -1;  // 2 * stage + prime
  uint32_t* tab = A1.scratch + (size_t)blockIdx.x * tab_stride;
  if (threadIdx.x == 0) next = atomicAdd(sync, 1u);
  __syncthreads();
  for (;;) {
    const uint64_t gt = next;
    if (gt >= T1 + U2) break;
    const bool st2 = gt >= T1;
    const uint64_t u = st2 ? gt - T1 : gt;
    const bool whole = !st2 || u < T2 - K2;
    const uint64_t j = whole ? u : T2 - K2 + (u - (T2 - K2)) / 2;  // tile (stage 2: also its stage-1 tile)
    const int hf = whole ? -1 : (int)((u - (T2 - K2)) & 1u);
    const ExpArgs& A = st2 ? A2 : A1;
    const int pi = j < A.pb[0].tiles ? 0 : 1;
    const ExpProblem& P = A.pb[pi];
    const uint64_t tile = pi == 0 ? j : j - A.pb[0].tiles;
    if (2 * (int)st2 + pi != loaded) {
      __syncthreads();
      if (st2) tc_load_operands<S2>(smem, P); else tc_load_operands<S1>(smem, P);
      tc_before_sync();
      __syncthreads();
      loaded = 2 * (int)st2 + pi;
    }
    if (st2) {
      if (threadIdx.x == 0) {
        uint32_t f;
        for (;;) {
          asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(f) : "l"(sync + 1 + j) : "memory");
          if (f) break;
          __nanosleep(256);
        }
      }
      __syncthreads();
      // y: written by another CTA of this launch
      tc_exp_tile<S2, FLB_TC_TRISQ_S2, true>(P, tile, A2.one, tab, whole ? sm2 : sm2h, phase, kLdGPU, hf);
    } else {
      tc_exp_tile<S1, FLB_TC_TRISQ_S1>(P, tile, A1.one, tab, sm1, phase);  // (single-buffered loads: measured)
    }
    __syncthreads();  // the tile's output rows are stored; the work rows are rewritten next
    if (threadIdx.x == 0) {
      if (!st2) {
        __threadfence();
        asm volatile("st.release.gpu.global.u32 [%0], %1;" :: "l"(sync + 1 + j), "r"(1u) : "memory");
      }
      next = atomicAdd(sync, 1u);
    }
    __syncthreads();
  }
  tc_cta_fini<COLS>(tmem_sh);
}

// debug: the product phase alone (t = a b, or a^2 when sq) for up to 128 elements -> t [count][2S]
template <int S, int SQ>
__global__ void __launch_bounds__(Cfg<S>::THREADS, 1) k_tc_debug_product(const uint32_t* a, const uint32_t* b, uint32_t* t,
                                                                  uint32_t count, int sq) {
  using C = Cfg<S>;
  extern __shared__ __align__(1024) uint8_t smem[];
  uint8_t* sA = smem + C::OFF_A;
  uint32_t* sW = reinterpret_cast<uint32_t*>(smem + C::OFF_W);
  tc_product<S, SQ>(src_arr(a, S, S, count), src_arr(b, S, S, count), sq != 0, sA, sW);
  __syncthreads();
  for (uint32_t i = threadIdx.x; i < count * 2 * S; i += C::THREADS) {
    const uint32_t e = i / (2 * S), w = i % (2 * S);
    t[i] = w < (uint32_t)S ? *reinterpret_cast<const uint32_t*>(sA + cm_off(e, 4u * w, C::KCH)) : sW[e * C::WROW + wpad<S>((int)w - S)];
  }
}

}  // namespace tc
}  // namespace flb
