// HMM forward on the 5th-generation tensor cores (tcgen05 + TMEM): the one
// step of the hot path that really is a dense GEMM (BASELINE north_star;
// SURVEY.md §8(a) A6c). Schedule S(s,i) = i (§5.2): the
// partition i of a group of 128 sequences is one [128 x 64] x [64 x 64] product
//     D[b][s] = sum_p alpha_{i-1}[b][p] * t_{p,s}
// followed by the emission / normalisation epilogue of Fig.11a (L472–L474).
//
// Warp-specialised CTA of kNG groups of 128 sequences (the MMA's M):
//   * the MMA warp (one elected lane) issues, per step and group, 12
//     tcgen05.mma.kind::f16 (M=128, N=64, K=16, A from TMEM) into that group's fp32 TMEM
//     accumulator (64 columns): alpha_hi x A_hi + alpha_hi x A_lo + alpha_lo x A_hi,
//     where x = x_hi + x_lo is a two-term bf16 split (the dropped lo x lo term is
//     ~2^-16 of a 2^-8 term: ~1e-7 relative per step, DESIGN.md §2 "HMM precision");
//     a tcgen05.commit arrives on the group's `full` mbarrier;
//   * four epilogue warps per group (warp w reads TMEM lane quarter w % 4), ONE
//     SEQUENCE PER THREAD over all 64 states: tcgen05.ld of the row, times e_s(x_i),
//     scaled by 1/R_{i-1} (the previous step's row sum, thread-local: lagged
//     scaling, log P = sum_i log R_i; packed fp32 pairs, FMUL2 / FADD2), split into
//     bf16 hi/lo and stored with tcgen05.st as the next A operand (TMEM, two bf16 per
//     column, K-major); all 128 threads arrive on the group's `ready` mbarrier of each
//     16-state K chunk as soon as it is stored.
// The groups' chains are independent, so the tensor pipe works on one group while
// the epilogue warps of the others run; no CTA-wide barrier inside the step loop
// (the row sum needs no cross-warp reduction when a thread owns a whole row).
// Within a group the steps overlap too: two accumulators alternate, and the epilogue signals
// each 16 states of the next operand as soon as they are in TMEM (one `ready` mbarrier per K
// chunk), so step i+1's MMAs for those K columns run while it still works on the rest.
// The transitions (B operand, hi/lo, 16 KB) live in shared memory; per group TMEM holds two
// fp32 accumulators (2 x 64 columns) and the next A operand alpha hi/lo (2 x 32 columns).
#include <algorithm>
#include <cstdint>
#include <cstdlib>
#include <cuda_bf16.h>
#include <cuda_runtime.h>

#include "dp_internal.h"

namespace dpk {
namespace {

constexpr int kM = 128;       // sequences per CTA (UMMA M)
constexpr int kS = 64;        // states (UMMA N and K)
constexpr int kCore = 128;    // bytes per 8x(16 B) core matrix
constexpr int kN2 = 2 * kS;    // N of the alpha_hi x [A_hi | A_lo] product

// K-major no-swizzle operand: core matrix (row group rg, k chunk kc) at
// (kc * row_groups + rg) * 128 bytes, rows of a core matrix 16 bytes apart.
__device__ __forceinline__ uint32_t op_offset(int row, int k, int row_groups) {
  return (uint32_t)(((k >> 3) * row_groups + (row >> 3)) * kCore + (row & 7) * 16 + (k & 7) * 2);
}

__device__ __forceinline__ uint64_t make_desc(uint32_t saddr, uint32_t lbo, uint32_t sbo) {
  uint64_t d = 0;
  d |= (uint64_t)((saddr >> 4) & 0x3fff);
  d |= (uint64_t)((lbo >> 4) & 0x3fff) << 16;
  d |= (uint64_t)((sbo >> 4) & 0x3fff) << 32;
  d |= (uint64_t)1 << 46;  // version (Blackwell)
  // base offset 0, lbo mode 0, layout type 0 = SWIZZLE_NONE
  return d;
}

// kind::f16 instruction descriptors: D f32, A/B bf16, both K-major, M = 128, N = 64 / 128
template <int N>
__host__ __device__ constexpr uint32_t idesc() { return (1u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(N >> 3) << 17) | ((uint32_t)(kM >> 4) << 24); }

template <int N>
__device__ __forceinline__ void mma_bf16(uint32_t tmem_d, uint64_t adesc, uint64_t bdesc, uint32_t accumulate) {
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "setp.ne.b32 p, %4, 0;\n\t"
      "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}\n"
      :
      : "r"(tmem_d), "l"(adesc), "l"(bdesc), "n"(idesc<N>()), "r"(accumulate));
}

// A from TMEM (the ".kind::f16 [d], [a], b_desc" form): A's rows in TMEM lanes, its K values
// packed two bf16 per 32-bit column (K-major), B from shared memory.
template <int N>
__device__ __forceinline__ void mma_bf16_ts(uint32_t tmem_d, uint32_t tmem_a, uint64_t bdesc, uint32_t accumulate) {
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "setp.ne.b32 p, %4, 0;\n\t"
      "tcgen05.mma.cta_group::1.kind::f16 [%0], [%1], %2, %3, p;\n\t}\n"
      :
      : "r"(tmem_d), "r"(tmem_a), "l"(bdesc), "n"(idesc<N>()), "r"(accumulate));
}

__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return (uint32_t)__cvta_generic_to_shared(p);
}

__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count));
}

__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
  asm volatile(
      "{\n\t.reg .pred done;\n\t"
      "WAIT_%=:\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 done, [%0], %1;\n\t"
      "@!done bra WAIT_%=;\n\t}\n" ::"r"(smem_u32(bar)),
      "r"(parity));
}

#define TMEM_LD16(taddr, r)                                                                                 \
  asm volatile(                                                                                             \
      "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];" \
      : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]),    \
        "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15]) \
      : "r"(taddr))

#ifndef HMM_TC_GROUPS
#define HMM_TC_GROUPS 1   // 1 / 2 / 4 groups: forward alone 1.07 / 1.26 / 2.17 ms, config-3 step 3.61 / 3.66 / 3.62 ms
#endif
constexpr int kNG = HMM_TC_GROUPS;         // sequence groups per CTA
constexpr int kEpiWarps = 4 * kNG;         // epilogue warps (4 per group: the TMEM lane quarters)
constexpr int kThreads = 32 * (kEpiWarps + 1);  // + the MMA warp
// TMEM columns per group: the fp32 accumulator (64), then alpha_hi and alpha_lo as the next A
// operand (64 bf16 = 32 columns each)
// two fp32 accumulators (steps alternate: step i+1's MMAs run while the epilogue still works on
// step i's row), then alpha_hi and alpha_lo as the next A operand (64 bf16 = 32 columns each)
constexpr int kColsAcc = 0, kColsAHi = 2 * kS, kColsALo = 2 * kS + kS / 2, kColsGroup = 4 * kS;
#ifndef HMM_TC_READY
#define HMM_TC_READY 16  // states per operand-ready signal (16 / 32 / 64: forward alone 0.842 / 0.858 / 0.899 ms)
#endif
constexpr int kReadyS = HMM_TC_READY;
constexpr int kChunks = kS / kReadyS;       // operand-ready signals per step
static_assert(kNG * kColsGroup <= 512, "TMEM: 512 columns per SM");

#define TMEM_ST8(taddr, w)                                                                      \
  asm volatile("tcgen05.st.sync.aligned.32x32b.x8.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8};" ::"r"(taddr), \
               "r"(w[0]), "r"(w[1]), "r"(w[2]), "r"(w[3]), "r"(w[4]), "r"(w[5]), "r"(w[6]), "r"(w[7]) : "memory")

struct TcSmem {
  alignas(128) uint8_t b_cat[kN2 * kS * 2];  // transitions (B operand): row n = s (A_hi) or 64 + s (A_lo), k = p
  alignas(16) float E[16][kS + 4];          // emission rows
  uint64_t full[kNG];                       // MMA -> epilogue: the group's accumulator is ready
  uint64_t ready[kNG][kChunks];             // epilogue -> MMA: states 16 kk .. 16 kk + 15 of the next operand stored
  uint32_t tmem_base;
  int tmax;
};

__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
  asm volatile("mbarrier.arrive.release.cta.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}

// Two bf16x2 words (hi, lo) with a + b = (hi.x + lo.x, hi.y + lo.y) to ~2^-16.
__device__ __forceinline__ void split2(float a, float b, uint32_t& hi, uint32_t& lo) {
  const __nv_bfloat162 h = __floats2bfloat162_rn(a, b);
  const float2 hf = __bfloat1622float2(h);
  const __nv_bfloat162 l = __floats2bfloat162_rn(a - hf.x, b - hf.y);
  hi = *reinterpret_cast<const uint32_t*>(&h);
  lo = *reinterpret_cast<const uint32_t*>(&l);
}

// Packed fp32 pairs (Blackwell FMUL2 / FADD2: one instruction per two states)
__device__ __forceinline__ uint64_t f2(float a, float b) {
  uint64_t r;
  asm("mov.b64 %0, {%1, %2};" : "=l"(r) : "f"(a), "f"(b));
  return r;
}
__device__ __forceinline__ uint64_t mul2(uint64_t a, uint64_t b) {
  uint64_t r;
  asm("mul.rn.f32x2 %0, %1, %2;" : "=l"(r) : "l"(a), "l"(b));
  return r;
}
__device__ __forceinline__ uint64_t add2(uint64_t a, uint64_t b) {
  uint64_t r;
  asm("add.rn.f32x2 %0, %1, %2;" : "=l"(r) : "l"(a), "l"(b));
  return r;
}
__device__ __forceinline__ uint64_t sub2(uint64_t a, uint64_t b) {
  uint64_t r;
  asm("sub.rn.f32x2 %0, %1, %2;" : "=l"(r) : "l"(a), "l"(b));
  return r;
}
// bf16x2 {lo: bf16(v.x), hi: bf16(v.y)}
__device__ __forceinline__ uint32_t cvt_bf2(uint64_t v) {
  uint32_t r;
  asm("{\n\t.reg .f32 a, b;\n\tmov.b64 {a, b}, %1;\n\tcvt.rn.bf16x2.f32 %0, b, a;\n\t}" : "=r"(r) : "l"(v));
  return r;
}
// (hi, lo) bf16x2 words with hi + lo = v to ~2^-16 (the two-term split, packed)
__device__ __forceinline__ void split2p(uint64_t v, uint32_t& hi, uint32_t& lo) {
  hi = cvt_bf2(v);
  const uint64_t hf = f2(__uint_as_float(hi << 16), __uint_as_float(hi & 0xffff0000u));
  lo = cvt_bf2(sub2(v, hf));
}

// Per step, with lagged scaling: alpha^_i = ((alpha^_{i-1} A) o e(x_i)) / R_{i-1},
// R_i = sum_s alpha^_i(s); then P(x) = prod_{i<=T} R_i and log P = sum log R_i. Dividing by the
// previous step's sum keeps R_i within the emission range because A is row-stochastic.
__global__ void __launch_bounds__(kThreads, 1) k_forward_tc(HmmArgs H) {
  extern __shared__ __align__(1024) uint8_t tc_raw[];
  TcSmem& sm = *reinterpret_cast<TcSmem*>(tc_raw);
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  const int S = H.S, K = H.K;

  // transitions: B[s][p] = t_{p,s} (K = p contiguous), split into bf16 hi/lo
  for (int q = tid; q < kS * kS; q += kThreads) {
    const int s = q / kS, pp = q % kS;
    const float v = (s < S && pp < S) ? H.A[pp * S + s] : 0.f;
    const __nv_bfloat16 hi = __float2bfloat16_rn(v);
    const __nv_bfloat16 lo = __float2bfloat16_rn(v - __bfloat162float(hi));
    *reinterpret_cast<__nv_bfloat16*>(sm.b_cat + op_offset(s, pp, kN2 / 8)) = hi;
    *reinterpret_cast<__nv_bfloat16*>(sm.b_cat + op_offset(kS + s, pp, kN2 / 8)) = lo;
  }
  for (int q = tid; q < 16 * (kS + 4); q += kThreads) {
    const int c = q / (kS + 4), s = q % (kS + 4);
    sm.E[c][s] = (c < K && s < S) ? H.E[s * K + c] : 0.f;
  }
  if (tid == 0) {
    for (int g = 0; g < kNG; ++g) {
      mbar_init(&sm.full[g], 1);
      for (int kk = 0; kk < kChunks; ++kk) mbar_init(&sm.ready[g][kk], 128);
    }
    sm.tmax = 0;
    asm volatile("fence.mbarrier_init.release.cluster;");
  }
  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(&sm.tmem_base)),
                 "n"(kNG * kColsGroup));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  // epilogue threads: group g, row b (TMEM lane 32 lq + lane)
  const bool epi = warp < kEpiWarps;
  const int g = epi ? warp >> 2 : 0, lq = warp & 3, b = 32 * lq + lane;
  const int64_t p = ((int64_t)blockIdx.x * kNG + g) * kM + b;
  const bool live = epi && p < H.n;
  const uint8_t* x = live ? H.x_cat + H.x_off[p] : nullptr;
  const int T = live ? (int)(H.x_off[p + 1] - H.x_off[p]) : 0;
  asm volatile("fence.proxy.async.shared::cta;");  // B (generic stores) -> the MMAs (async proxy)
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;");
  const uint32_t tmem = sm.tmem_base;
  if (T > 0) atomicMax(&sm.tmax, T);
  __syncthreads();
  const int Tmax = sm.tmax;

  if (!epi) {  // ------------------------------------------------------------ the MMA warp
    if (lane == 0) {
      const uint64_t dB = make_desc(smem_u32(sm.b_cat), (kN2 / 8) * kCore, kCore);
      // A_lo: rows n = 64 .. 127 of the B buffer (8 row groups further on)
      const uint64_t dB_lo = make_desc(smem_u32(sm.b_cat) + (kS / 8) * kCore, (kN2 / 8) * kCore, kCore);
      // D_g = a_hi*A_hi + a_hi*A_lo + a_lo*A_hi: three N = 64 products into the same 64 columns;
      // K = 64 in 4 steps of 16.
      // Descriptor address fields count 16-byte units: a K step of 16 is two core matrices.
      for (int i = 2; i <= Tmax; ++i) {
        for (int q = 0; q < kNG; ++q) {
          const uint32_t td = tmem + (uint32_t)(q * kColsGroup + kColsAcc + (i & 1) * kS);
          const uint32_t ta_hi = tmem + (uint32_t)(q * kColsGroup + kColsAHi);
          const uint32_t ta_lo = tmem + (uint32_t)(q * kColsGroup + kColsALo);
#pragma unroll
          for (int kk = 0; kk < kS / 16; ++kk) {  // a K step of 16 bf16: 8 TMEM columns of A, issued as
            if ((16 * kk) % kReadyS == 0) {       // soon as the epilogue stored them
              mbar_wait(&sm.ready[q][16 * kk / kReadyS], (uint32_t)(i - 2) & 1u);
              asm volatile("tcgen05.fence::after_thread_sync;");
            }
            const uint64_t kb = (uint64_t)(2 * kk * (kN2 / 8) * kCore >> 4);
            mma_bf16_ts<kS>(td, ta_hi + 8 * kk, dB + kb, kk > 0);  // a_hi x A_hi
            mma_bf16_ts<kS>(td, ta_hi + 8 * kk, dB_lo + kb, 1);    // a_hi x A_lo
            mma_bf16_ts<kS>(td, ta_lo + 8 * kk, dB + kb, 1);       // a_lo x A_hi
          }
          asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(
              smem_u32(&sm.full[q])));
        }
      }
    }
  } else {  // -------------------------------------------------------------- epilogue warps
    const uint32_t trow = tmem + ((uint32_t)(lq * 32) << 16) + (uint32_t)(g * kColsGroup);
    // 16 values of alpha^ (states k0 .. k0 + 15) into this row of the group's TMEM A operand
    auto store16 = [&](int k0, const float* v) {
      uint32_t hw[8], lw[8];
#pragma unroll
      for (int q = 0; q < 8; ++q) split2(v[2 * q], v[2 * q + 1], hw[q], lw[q]);
      TMEM_ST8(trow + kColsAHi + k0 / 2, hw);
      TMEM_ST8(trow + kColsALo + k0 / 2, lw);
    };
    double prod = 1.0;  // prod of R_i, renormalised: P = prod * 2^pexp
    int pexp = 0;
    float R = 0.f;      // this row's sum of the previous step
    // i = 1: alpha^_1(s) = pi_s e_s(x_1) (no scaling)
    {
      const int c = T > 0 ? x[0] : 0;
#pragma unroll
      for (int k0 = 0; k0 < kS; k0 += 16) {
        float v[16];
#pragma unroll
        for (int q = 0; q < 16; ++q) {
          const int s = k0 + q;
          v[q] = (s < S && T > 0) ? H.pi[s] * sm.E[c][s] : 0.f;
          R += v[q];
        }
        store16(k0, v);
      }
    }
    asm volatile("tcgen05.wait::st.sync.aligned;");
    asm volatile("tcgen05.fence::before_thread_sync;");
#pragma unroll
    for (int kk = 0; kk < kChunks; ++kk) mbar_arrive(&sm.ready[g][kk]);
    uint4 xs = make_uint4(0, 0, 0, 0);
    for (int i = 2; i <= Tmax; ++i) {
      const float inv = R > 0.f ? 1.f / R : 0.f;
      if (i - 1 <= T) {
        prod *= (double)R;
        if ((i & 15) == 0) {  // keep the product normal: P = prod * 2^pexp
          int e2;
          prod = frexp(prod, &e2);
          pexp += e2;
        }
      }
      if (((i - 2) & 15) == 0 && i - 1 < T) {
        uint8_t tmp[16];
#pragma unroll
        for (int u = 0; u < 16; ++u) tmp[u] = (i - 1 + u < T) ? x[i - 1 + u] : 0;
        xs = *reinterpret_cast<uint4*>(tmp);
      }
      const int sh = (i - 2) & 15;
      const uint32_t word = sh < 4 ? xs.x : sh < 8 ? xs.y : sh < 12 ? xs.z : xs.w;
      const float* er = &sm.E[(word >> (8 * (sh & 3))) & 0xff][0];
      mbar_wait(&sm.full[g], (uint32_t)(i - 2) & 1u);
      asm volatile("tcgen05.fence::after_thread_sync;");
      uint64_t tot2 = 0;  // (+0.f, +0.f)
      // a finished row keeps storing a zero operand (the .sync.aligned stores are warp-uniform
      // calls): its scale is 0 (the accumulator and the emissions are finite)
      const float sc = i > T ? 0.f : inv;
      const uint64_t inv2 = f2(sc, sc);
      uint32_t r[kS];  // the row: 64 accumulators, four loads and one wait
      const uint32_t taddr = trow + kColsAcc + (i & 1) * kS;
      TMEM_LD16(taddr, r);
      TMEM_LD16(taddr + 16, (r + 16));
      TMEM_LD16(taddr + 32, (r + 32));
      TMEM_LD16(taddr + 48, (r + 48));
      asm volatile("tcgen05.wait::ld.sync.aligned;");
      // per pair of states: (e * inv), times the accumulator, into the row sum, split to bf16
      // hi / lo — 8 instructions per two states (FMUL2, FMUL2, FADD2, F2FP, 2 unpacks, FADD2, F2FP)
#pragma unroll
      for (int k0 = 0; k0 < kS; k0 += 16) {
        const float4* e4 = reinterpret_cast<const float4*>(er + k0);
        const float4 e0 = e4[0], e1 = e4[1], e2 = e4[2], e3 = e4[3];
        const uint64_t ev[8] = {f2(e0.x, e0.y), f2(e0.z, e0.w), f2(e1.x, e1.y), f2(e1.z, e1.w),
                                f2(e2.x, e2.y), f2(e2.z, e2.w), f2(e3.x, e3.y), f2(e3.z, e3.w)};
        uint32_t hw[8], lw[8];
#pragma unroll
        for (int q = 0; q < 8; ++q) {
          const uint64_t v = mul2(f2(__uint_as_float(r[k0 + 2 * q]), __uint_as_float(r[k0 + 2 * q + 1])),
                                  mul2(ev[q], inv2));
          tot2 = add2(tot2, v);
          split2p(v, hw[q], lw[q]);
        }
        TMEM_ST8(trow + kColsAHi + k0 / 2, hw);
        TMEM_ST8(trow + kColsALo + k0 / 2, lw);
        // these states of the next operand are in TMEM: the next step's K chunks may start
        if ((k0 + 16) % kReadyS == 0) {
          asm volatile("tcgen05.wait::st.sync.aligned;");
          asm volatile("tcgen05.fence::before_thread_sync;");
          mbar_arrive(&sm.ready[g][k0 / kReadyS]);
        }
      }
      if (i <= T) {
        float t0, t1;
        asm("mov.b64 {%0, %1}, %2;" : "=f"(t0), "=f"(t1) : "l"(tot2));
        R = t0 + t1;
      }
    }
    if (Tmax >= 1 && Tmax <= T) prod *= (double)R;  // R_T of the sequences that run to the end
    if (live) H.ll_out[p] = T == 0 ? 0.f : (float)(log(prod) + (double)pexp * 0.69314718055994530942);
  }
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  if (warp == 0) {
    asm volatile("tcgen05.fence::after_thread_sync;");
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "n"(kNG * kColsGroup));
  }
}

}  // namespace

bool hmm_forward_tc_supported(int S) { return S <= kS; }

cudaError_t hmm_forward_tc(const HmmArgs& H, cudaStream_t s, int64_t* launches) {
  if (H.n == 0) return cudaSuccess;
  // The step is a latency chain (MMA -> epilogue -> MMA); the shared memory a CTA reserves decides
  // how many of a concurrent kernel's CTAs (Viterbi) may share its SM (tc_smem_kb).
  const size_t need = sizeof(TcSmem) + 1024;
  const size_t smem = std::max(need, (size_t)(H.tc_smem_kb >= 0 ? H.tc_smem_kb : 0) * 1024);
  cudaError_t e = cudaFuncSetAttribute(k_forward_tc, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  ++*launches;
  k_forward_tc<<<(unsigned)((H.n + kNG * kM - 1) / (kNG * kM)), kThreads, smem, s>>>(H);
  return cudaGetLastError();
}

}  // namespace dpk
