// HMM forward and Viterbi on the derived schedule S(s,i) = i (§5.2
// L467–L472: "our schedule can only be S_forward(s,i) = i").
// Partition i holds the S cells F(., i); the window is one partition (§4.8).
//
// B200 design (SIMT, round 1): one warp per sequence, lane l owns states l and
// l + 32 (S <= 64). The column of the transition matrix for each owned state
// (64 + 64 values) stays in registers for the whole sequence, the previous
// partition's S values are broadcast from shared memory, so one step is
// 128 FFMA (forward) or 128 VIADDMNMX (Viterbi) per lane with no global traffic.
//
// Forward (Fig.11a; DESIGN.md R-HMM-FWD): begin state with
// transitions pi, tau == 1. Probabilities are kept in scaled linear space
// (one of the representations §3.2 L222–L225 allows): alpha_i = a_i / c_i with
// c_i = sum_s a_i(s), log P(x) = sum_i log c_i accumulated in fp64.
// Viterbi (max-variant, L463–L464; DESIGN.md R-VIT): int32 milli-bit scores,
// exact integer arithmetic. The predecessor argmax with lowest-index ties uses
// packed keys key(p) = V(p) * 64 + (63 - p), so one VIADDMNMX per (p, s) yields
// both the max and the argmax; V is renormalised by its max every step
// (integer offset kept in int64) so keys never overflow.
#include <cstdint>
#include <cuda_runtime.h>

#include "dp_internal.h"

namespace dpk {
namespace {

constexpr int kMaxS = 64;
constexpr int kMaxK = 16;

__device__ __forceinline__ float warp_sum(float v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
  return v;
}
__device__ __forceinline__ int warp_max(int v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v = max(v, __shfl_xor_sync(0xffffffffu, v, o));
  return v;
}

__global__ void __launch_bounds__(kWarps * 32, 1) k_forward(HmmArgs H) {
  __shared__ __align__(16) float alpha[kWarps][kMaxS];
  __shared__ float Es[kMaxS * kMaxK];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int S = H.S, K = H.K;
  for (int q = threadIdx.x; q < kMaxS * kMaxK; q += blockDim.x) {
    const int s = q / kMaxK, c = q % kMaxK;
    Es[q] = (s < S && c < K) ? H.E[s * K + c] : 0.f;
  }
  __syncthreads();
  const int64_t p = (int64_t)blockIdx.x * kWarps + warp;
  if (p >= H.n) return;
  const int s0 = lane, s1 = lane + 32;
  float a0[kMaxS], a1[kMaxS];
#pragma unroll
  for (int q = 0; q < kMaxS; ++q) {
    a0[q] = (q < S && s0 < S) ? H.A[q * S + s0] : 0.f;
    a1[q] = (q < S && s1 < S) ? H.A[q * S + s1] : 0.f;
  }
  const uint8_t* x = H.x_cat + H.x_off[p];
  const int T = (int)(H.x_off[p + 1] - H.x_off[p]);
  if (T == 0) {
    if (lane == 0) H.ll_out[p] = 0.f;
    return;
  }
  double ll = 0.0;
  // i = 1: a(s) = pi_s e_s(x_1)
  int c = x[0];
  float v0 = (s0 < S) ? H.pi[s0] * Es[s0 * kMaxK + c] : 0.f;
  float v1 = (s1 < S) ? H.pi[s1] * Es[s1 * kMaxK + c] : 0.f;
  float tot = warp_sum(v0 + v1);
  ll += log((double)tot);
  float inv = 1.f / tot;
  alpha[warp][s0] = v0 * inv;
  alpha[warp][s1] = v1 * inv;
  __syncwarp();
  int cn = (T > 1) ? x[1] : 0;
  for (int i = 2; i <= T; ++i) {
    c = cn;
    if (i < T) cn = x[i];  // prefetch the next symbol
    float acc0[4] = {0.f, 0.f, 0.f, 0.f}, acc1[4] = {0.f, 0.f, 0.f, 0.f};
    const float4* al = reinterpret_cast<const float4*>(alpha[warp]);
#pragma unroll
    for (int q4 = 0; q4 < kMaxS / 4; ++q4) {
      const float4 v = al[q4];
      acc0[0] = fmaf(v.x, a0[4 * q4 + 0], acc0[0]);
      acc0[1] = fmaf(v.y, a0[4 * q4 + 1], acc0[1]);
      acc0[2] = fmaf(v.z, a0[4 * q4 + 2], acc0[2]);
      acc0[3] = fmaf(v.w, a0[4 * q4 + 3], acc0[3]);
      acc1[0] = fmaf(v.x, a1[4 * q4 + 0], acc1[0]);
      acc1[1] = fmaf(v.y, a1[4 * q4 + 1], acc1[1]);
      acc1[2] = fmaf(v.z, a1[4 * q4 + 2], acc1[2]);
      acc1[3] = fmaf(v.w, a1[4 * q4 + 3], acc1[3]);
    }
    v0 = ((acc0[0] + acc0[1]) + (acc0[2] + acc0[3])) * Es[s0 * kMaxK + c];
    v1 = ((acc1[0] + acc1[1]) + (acc1[2] + acc1[3])) * Es[s1 * kMaxK + c];
    tot = warp_sum(v0 + v1);
    ll += log((double)tot);
    inv = 1.f / tot;
    __syncwarp();
    alpha[warp][s0] = v0 * inv;
    alpha[warp][s1] = v1 * inv;
    __syncwarp();
  }
  if (lane == 0) H.ll_out[p] = (float)ll;
}

constexpr int kNegKey = -(1 << 30);

__global__ void __launch_bounds__(kWarps * 32, 1) k_viterbi(HmmArgs H) {
  __shared__ __align__(16) int key[kWarps][kMaxS];
  __shared__ int Es[kMaxS * kMaxK];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int S = H.S, K = H.K;
  for (int q = threadIdx.x; q < kMaxS * kMaxK; q += blockDim.x) {
    const int s = q / kMaxK, c = q % kMaxK;
    Es[q] = (s < S && c < K) ? H.lE[s * K + c] : 0;
  }
  __syncthreads();
  const int64_t p = (int64_t)blockIdx.x * kWarps + warp;
  if (p >= H.n) return;
  const int s0 = lane, s1 = lane + 32;
  const bool ok0 = s0 < S, ok1 = s1 < S;
  int la0[kMaxS], la1[kMaxS];  // transition scores x 64 (key units)
#pragma unroll
  for (int q = 0; q < kMaxS; ++q) {
    la0[q] = (q < S && ok0) ? H.lA[q * S + s0] * 64 : 0;
    la1[q] = (q < S && ok1) ? H.lA[q * S + s1] * 64 : 0;
  }
  const uint8_t* x = H.x_cat + H.x_off[p];
  const int T = (int)(H.x_off[p + 1] - H.x_off[p]);
  if (T == 0) {
    if (lane == 0) { H.vit_out[p] = 0; if (H.final_state) H.final_state[p] = -1; }
    return;
  }
  uint8_t* bp = H.bp ? H.bp + (p * H.max_len) * kMaxS : nullptr;
  // i = 1: V(s) = lpi_s + lE[s, x_1]
  int c = x[0];
  int V0 = ok0 ? H.lpi[s0] + Es[s0 * kMaxK + c] : kNegKey;
  int V1 = ok1 ? H.lpi[s1] + Es[s1 * kMaxK + c] : kNegKey;
  int m = warp_max(max(V0, V1));
  int64_t off = m;
  V0 -= m; V1 -= m;
  key[warp][s0] = ok0 ? V0 * 64 + (63 - s0) : kNegKey;
  key[warp][s1] = ok1 ? V1 * 64 + (63 - s1) : kNegKey;
  __syncwarp();
  int cn = (T > 1) ? x[1] : 0;
  for (int i = 2; i <= T; ++i) {
    c = cn;
    if (i < T) cn = x[i];
    int b0[4] = {INT32_MIN, INT32_MIN, INT32_MIN, INT32_MIN}, b1[4] = {INT32_MIN, INT32_MIN, INT32_MIN, INT32_MIN};
    const int4* kv = reinterpret_cast<const int4*>(key[warp]);
#pragma unroll
    for (int q4 = 0; q4 < kMaxS / 4; ++q4) {
      const int4 v = kv[q4];
      b0[0] = __viaddmax_s32(v.x, la0[4 * q4 + 0], b0[0]);
      b0[1] = __viaddmax_s32(v.y, la0[4 * q4 + 1], b0[1]);
      b0[2] = __viaddmax_s32(v.z, la0[4 * q4 + 2], b0[2]);
      b0[3] = __viaddmax_s32(v.w, la0[4 * q4 + 3], b0[3]);
      b1[0] = __viaddmax_s32(v.x, la1[4 * q4 + 0], b1[0]);
      b1[1] = __viaddmax_s32(v.y, la1[4 * q4 + 1], b1[1]);
      b1[2] = __viaddmax_s32(v.z, la1[4 * q4 + 2], b1[2]);
      b1[3] = __viaddmax_s32(v.w, la1[4 * q4 + 3], b1[3]);
    }
    const int k0 = max(max(b0[0], b0[1]), max(b0[2], b0[3]));
    const int k1 = max(max(b1[0], b1[1]), max(b1[2], b1[3]));
    // key = V(p)*64 + (63-p) + lA*64  ->  floor(key / 64) = V(p) + lA, low 6 bits = 63 - argmax
    V0 = ok0 ? (k0 >> 6) + Es[s0 * kMaxK + c] : kNegKey;
    V1 = ok1 ? (k1 >> 6) + Es[s1 * kMaxK + c] : kNegKey;
    if (bp) {
      if (ok0) bp[(int64_t)(i - 1) * kMaxS + s0] = (uint8_t)(63 - (k0 & 63));
      if (ok1) bp[(int64_t)(i - 1) * kMaxS + s1] = (uint8_t)(63 - (k1 & 63));
    }
    m = warp_max(max(V0, V1));
    off += m;
    V0 -= m; V1 -= m;
    __syncwarp();
    key[warp][s0] = ok0 ? V0 * 64 + (63 - s0) : kNegKey;
    key[warp][s1] = ok1 ? V1 * 64 + (63 - s1) : kNegKey;
    __syncwarp();
  }
  // best final state: max V, lowest index on ties -> max of V*64 + (63 - s)
  const int fk = warp_max(max(key[warp][s0], key[warp][s1]));
  if (lane == 0) {
    H.vit_out[p] = (int32_t)(off + (fk >> 6));
    if (H.final_state) H.final_state[p] = 63 - (fk & 63);
  }
}

__global__ void k_viterbi_tb(HmmArgs H, int64_t first, int64_t count, uint8_t* out, int64_t stride,
                             int32_t* out_len) {
  const int64_t q = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (q >= count) return;
  const int64_t p = first + q;
  const int T = (int)(H.x_off[p + 1] - H.x_off[p]);
  if (T > stride) { out_len[q] = -1; return; }
  const uint8_t* bp = H.bp + (p * H.max_len) * kMaxS;
  uint8_t* o = out + q * stride;
  int s = H.final_state[p];
  for (int i = T; i >= 1; --i) {
    o[i - 1] = (uint8_t)s;
    if (i > 1) s = bp[(int64_t)(i - 1) * kMaxS + s];
  }
  out_len[q] = T;
}

}  // namespace

cudaError_t hmm_forward(const HmmArgs& H, cudaStream_t s, int64_t* launches) {
  if (H.n == 0) return cudaSuccess;
  ++*launches;
  k_forward<<<(unsigned)((H.n + kWarps - 1) / kWarps), kWarps * 32, 0, s>>>(H);
  return cudaGetLastError();
}

cudaError_t hmm_viterbi(const HmmArgs& H, cudaStream_t s, int64_t* launches) {
  if (H.n == 0) return cudaSuccess;
  ++*launches;
  k_viterbi<<<(unsigned)((H.n + kWarps - 1) / kWarps), kWarps * 32, 0, s>>>(H);
  return cudaGetLastError();
}

cudaError_t hmm_viterbi_traceback(const HmmArgs& H, int64_t first, int64_t count, uint8_t* out, int64_t stride,
                                  int32_t* out_len, cudaStream_t s, int64_t* launches) {
  if (count == 0) return cudaSuccess;
  ++*launches;
  k_viterbi_tb<<<(unsigned)((count + 127) / 128), 128, 0, s>>>(H, first, count, out, stride, out_len);
  return cudaGetLastError();
}

}  // namespace dpk
