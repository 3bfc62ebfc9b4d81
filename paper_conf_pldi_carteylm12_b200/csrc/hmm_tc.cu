// HMM forward on the 5th-generation tensor cores (tcgen05 + TMEM): the one
// step of the hot path that really is a dense GEMM (BASELINE north_star;
// SURVEY.md §8(a) A6c). Schedule S(s,i) = i (§5.2): the
// partition i of 128 sequences is one [128 x 64] x [64 x 64] product
//     D[b][s] = sum_p alpha_{i-1}[b][p] * t_{p,s}
// followed by the emission / normalisation epilogue of Fig.11a (L472–L474).
//
// One CTA = 128 sequences (the MMA's M), 4 warps. Thread b owns sequence b and
// TMEM lane b. Per step:
//   * thread 0 issues 12 tcgen05.mma.kind::f16 (M=128, N=64, K=16) into the
//     fp32 TMEM accumulator: alpha_hi*A_hi + alpha_hi*A_lo + alpha_lo*A_hi,
//     where x = x_hi + x_lo is a two-term bf16 split (product error ~2^-16 of
//     a 2^-8 term: ~1e-7 relative per step);
//   * tcgen05.commit arrives on an mbarrier; all threads wait on it, read
//     their 64 columns with tcgen05.ld, multiply by e_s(x_i), normalise by the
//     row sum c_i (log P = sum_i log c_i, fp64), split into bf16 hi/lo and
//     store them in shared memory in the canonical K-major no-swizzle UMMA
//     layout (8x16-byte core matrices) for the next step.
// Operands live in shared memory (alpha hi/lo 2 x 16 KB, transitions hi/lo
// 2 x 8 KB); the accumulator lives in TMEM (64 columns).
#include <cstdint>
#include <cuda_bf16.h>
#include <cuda_runtime.h>

#include "dp_internal.h"

namespace dpk {
namespace {

constexpr int kM = 128;       // sequences per CTA (UMMA M)
constexpr int kS = 64;        // states (UMMA N and K)
constexpr int kCore = 128;    // bytes per 8x(16 B) core matrix
constexpr int kTmemCols = 64;

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

// kind::f16 instruction descriptor: D f32, A/B bf16, both K-major, N = 64, M = 128
constexpr uint32_t kIdesc = (1u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(kS >> 3) << 17) | ((uint32_t)(kM >> 4) << 24);

__device__ __forceinline__ void mma_bf16(uint32_t tmem_d, uint64_t adesc, uint64_t bdesc, uint32_t accumulate) {
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "setp.ne.b32 p, %4, 0;\n\t"
      "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}\n"
      :
      : "r"(tmem_d), "l"(adesc), "l"(bdesc), "r"(kIdesc), "r"(accumulate));
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

struct TcSmem {
  alignas(128) uint8_t a_hi[kM * kS * 2];   // alpha (A operand), K-major core matrices
  alignas(128) uint8_t a_lo[kM * kS * 2];
  alignas(128) uint8_t b_hi[kS * kS * 2];   // transitions (B operand): row = s (N), k = p
  alignas(128) uint8_t b_lo[kS * kS * 2];
  alignas(16) float E[16][kS + 4];          // emission rows, padded against bank conflicts
  uint64_t bar;
  uint32_t tmem_base;
};

// bf16 pair split: v = hi + lo with hi = bf16(v), lo = bf16(v - hi)
__device__ __forceinline__ void split_bf16(float v, __nv_bfloat16& hi, __nv_bfloat16& lo) {
  hi = __float2bfloat16_rn(v);
  lo = __float2bfloat16_rn(v - __bfloat162float(hi));
}

__global__ void __launch_bounds__(kM, 1) k_forward_tc(HmmArgs H) {
  extern __shared__ __align__(1024) uint8_t tc_raw[];
  TcSmem& sm = *reinterpret_cast<TcSmem*>(tc_raw);
  const int tid = threadIdx.x, warp = tid >> 5;
  const int S = H.S, K = H.K;
  const int64_t p = (int64_t)blockIdx.x * kM + tid;
  const bool live = p < H.n;

  // transitions: B[s][p] = t_{p,s} (K = p contiguous), split into bf16 hi/lo
  for (int q = tid; q < kS * kS; q += kM) {
    const int s = q / kS, pp = q % kS;
    const float v = (s < S && pp < S) ? H.A[pp * S + s] : 0.f;
    __nv_bfloat16 hi, lo;
    split_bf16(v, hi, lo);
    const uint32_t off = op_offset(s, pp, kS / 8);
    *reinterpret_cast<__nv_bfloat16*>(sm.b_hi + off) = hi;
    *reinterpret_cast<__nv_bfloat16*>(sm.b_lo + off) = lo;
  }
  for (int q = tid; q < 16 * (kS + 4); q += kM) {
    const int c = q / (kS + 4), s = q % (kS + 4);
    sm.E[c][s] = (c < K && s < S) ? H.E[s * K + c] : 0.f;
  }
  if (tid == 0) {
    mbar_init(&sm.bar, 1);
    asm volatile("fence.mbarrier_init.release.cluster;");
  }
  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(&sm.tmem_base)),
                 "n"(kTmemCols));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  asm volatile("fence.proxy.async.shared::cta;");
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;");
  const uint32_t tmem = sm.tmem_base;

  const uint8_t* x = live ? H.x_cat + H.x_off[p] : nullptr;
  const int T = live ? (int)(H.x_off[p + 1] - H.x_off[p]) : 0;
  int Tmax = T;
  // the CTA runs to its longest sequence
  {
    __shared__ int tmax_s;
    if (tid == 0) tmax_s = 0;
    __syncthreads();
    atomicMax(&tmax_s, T);
    __syncthreads();
    Tmax = tmax_s;
  }
  float alpha[kS];
  double ll = 0.0;
  // i = 1: a(s) = pi_s e_s(x_1)
  {
    const int c = T > 0 ? x[0] : 0;
    float tot = 0.f;
#pragma unroll
    for (int s = 0; s < kS; ++s) {
      alpha[s] = (s < S && T > 0) ? H.pi[s] * sm.E[c][s] : 0.f;
      tot += alpha[s];
    }
    const float inv = tot > 0.f ? 1.f / tot : 0.f;
    if (T > 0) ll = log((double)tot);
#pragma unroll
    for (int s = 0; s < kS; ++s) alpha[s] *= inv;
  }
  const uint32_t a_hi = smem_u32(sm.a_hi), a_lo = smem_u32(sm.a_lo);
  const uint32_t b_hi = smem_u32(sm.b_hi), b_lo = smem_u32(sm.b_lo);
  const uint32_t taddr = tmem + ((uint32_t)(warp * 32) << 16);  // this warp's 32 TMEM lanes
  uint32_t parity = 0;
  uint4 xs = make_uint4(0, 0, 0, 0);
  for (int i = 2; i <= Tmax; ++i) {
    // alpha_{i-1} -> shared memory (bf16 hi/lo, K-major core matrices)
#pragma unroll
    for (int kc = 0; kc < kS / 8; ++kc) {
      uint32_t hw[4], lw[4];
#pragma unroll
      for (int q = 0; q < 4; ++q) {
        __nv_bfloat16 h0, l0, h1, l1;
        split_bf16(alpha[kc * 8 + 2 * q], h0, l0);
        split_bf16(alpha[kc * 8 + 2 * q + 1], h1, l1);
        hw[q] = (uint32_t)__bfloat16_as_ushort(h0) | ((uint32_t)__bfloat16_as_ushort(h1) << 16);
        lw[q] = (uint32_t)__bfloat16_as_ushort(l0) | ((uint32_t)__bfloat16_as_ushort(l1) << 16);
      }
      const uint32_t off = op_offset(tid, kc * 8, kM / 8);
      *reinterpret_cast<uint4*>(sm.a_hi + off) = make_uint4(hw[0], hw[1], hw[2], hw[3]);
      *reinterpret_cast<uint4*>(sm.a_lo + off) = make_uint4(lw[0], lw[1], lw[2], lw[3]);
    }
    asm volatile("fence.proxy.async.shared::cta;");
    asm volatile("tcgen05.fence::before_thread_sync;");
    __syncthreads();
    if (tid == 0) {
      asm volatile("tcgen05.fence::after_thread_sync;");
      // D = a_hi*b_hi + a_hi*b_lo + a_lo*b_hi, K = 64 in 4 steps of 16
#pragma unroll
      for (int kk = 0; kk < kS / 16; ++kk) {
        const uint32_t ka = (uint32_t)(2 * kk) * (kM / 8) * kCore;  // two k chunks per MMA
        const uint32_t kb = (uint32_t)(2 * kk) * (kS / 8) * kCore;
        mma_bf16(tmem, make_desc(a_hi + ka, (kM / 8) * kCore, kCore), make_desc(b_hi + kb, (kS / 8) * kCore, kCore),
                 kk > 0);
      }
#pragma unroll
      for (int kk = 0; kk < kS / 16; ++kk) {
        const uint32_t ka = (uint32_t)(2 * kk) * (kM / 8) * kCore;
        const uint32_t kb = (uint32_t)(2 * kk) * (kS / 8) * kCore;
        mma_bf16(tmem, make_desc(a_hi + ka, (kM / 8) * kCore, kCore), make_desc(b_lo + kb, (kS / 8) * kCore, kCore), 1);
      }
#pragma unroll
      for (int kk = 0; kk < kS / 16; ++kk) {
        const uint32_t ka = (uint32_t)(2 * kk) * (kM / 8) * kCore;
        const uint32_t kb = (uint32_t)(2 * kk) * (kS / 8) * kCore;
        mma_bf16(tmem, make_desc(a_lo + ka, (kM / 8) * kCore, kCore), make_desc(b_hi + kb, (kS / 8) * kCore, kCore), 1);
      }
      asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(
          smem_u32(&sm.bar)));
    }
    // next symbol (prefetched 16 at a time) while the MMAs run
    if (((i - 2) & 15) == 0 && i - 1 < T) {
      uint8_t tmp[16];
#pragma unroll
      for (int q = 0; q < 16; ++q) tmp[q] = (i - 1 + q < T) ? x[i - 1 + q] : 0;
      xs = *reinterpret_cast<uint4*>(tmp);
    }
    const int sh = (i - 2) & 15;
    const uint32_t word = sh < 4 ? xs.x : sh < 8 ? xs.y : sh < 12 ? xs.z : xs.w;
    const int c = (word >> (8 * (sh & 3))) & 0xff;
    mbar_wait(&sm.bar, parity);
    parity ^= 1;
    asm volatile("tcgen05.fence::after_thread_sync;");
    uint32_t r[kS];
    TMEM_LD16(taddr + 0, (&r[0]));
    TMEM_LD16(taddr + 16, (&r[16]));
    TMEM_LD16(taddr + 32, (&r[32]));
    TMEM_LD16(taddr + 48, (&r[48]));
    asm volatile("tcgen05.wait::ld.sync.aligned;");
    if (i <= T) {
      const float4* er = reinterpret_cast<const float4*>(sm.E[c]);
      float tot = 0.f;
#pragma unroll
      for (int q4 = 0; q4 < kS / 4; ++q4) {
        const float4 e = er[q4];
        alpha[4 * q4 + 0] = __uint_as_float(r[4 * q4 + 0]) * e.x;
        alpha[4 * q4 + 1] = __uint_as_float(r[4 * q4 + 1]) * e.y;
        alpha[4 * q4 + 2] = __uint_as_float(r[4 * q4 + 2]) * e.z;
        alpha[4 * q4 + 3] = __uint_as_float(r[4 * q4 + 3]) * e.w;
        tot += (alpha[4 * q4 + 0] + alpha[4 * q4 + 1]) + (alpha[4 * q4 + 2] + alpha[4 * q4 + 3]);
      }
      const float inv = tot > 0.f ? 1.f / tot : 0.f;
      ll += log((double)tot);
#pragma unroll
      for (int s = 0; s < kS; ++s) alpha[s] *= inv;
    }
  }
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  if (warp == 0) {
    asm volatile("tcgen05.fence::after_thread_sync;");
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "n"(kTmemCols));
  }
  if (live) H.ll_out[p] = T == 0 ? 0.f : (float)ll;
}

}  // namespace

bool hmm_forward_tc_supported(int S) { return S <= kS && getenv("DP_HMM_SIMT") == nullptr; }

cudaError_t hmm_forward_tc(const HmmArgs& H, cudaStream_t s, int64_t* launches) {
  if (H.n == 0) return cudaSuccess;
  const size_t smem = sizeof(TcSmem) + 1024;
  cudaError_t e = cudaFuncSetAttribute(k_forward_tc, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  ++*launches;
  k_forward_tc<<<(unsigned)((H.n + kM - 1) / kM), kM, smem, s>>>(H);
  return cudaGetLastError();
}

}  // namespace dpk
