// HMM forward and Viterbi on the derived schedule S(s,i) = i (§5.2
// L467–L472: "our schedule can only be S_forward(s,i) = i").
// Partition i holds the S cells F(., i); the window is one partition (§4.8).
//
// B200 design (SIMT): one warp carries NS sequences, lane l owns states l and
// l + 32 (S <= 64). The columns of the transition matrix for the two owned
// states (64 + 64 values) stay in registers for the whole batch and are
// reused by all NS sequences; the previous partition of each sequence is
// broadcast from shared memory by LDS.128. One step is 128 x NS FFMA (forward)
// or VIADDMNMX (Viterbi) per lane, with NS independent chains to hide the
// per-step reduction latency. NS is picked so the batch fits in one wave.
//
// Forward (Fig.11a; DESIGN.md R-HMM-FWD): begin state with
// transitions pi, tau == 1. Probabilities are kept in scaled linear space
// (one of the representations §3.2 L222–L225 allows): alpha_i = a_i / c_i with
// c_i = sum_s a_i(s); log P(x) = sum_i log c_i, the c_i multiplied in fp32 and
// folded into an fp64 log sum whenever the product leaves [2^-60, 2^60].
// Viterbi (max-variant, L463–L464; DESIGN.md R-VIT): int32 milli-bit scores,
// exact integer arithmetic. The predecessor argmax with lowest-index ties uses
// packed keys key(p) = V(p) * 64 + (63 - p), so one VIADDMNMX per (p, s) yields
// both the max and the argmax; V is renormalised by its max every 32 steps
// (exact integer offset kept in int64) so keys never overflow.
#include <algorithm>
#include <cstdint>
#include <cstdlib>
#include <cuda_runtime.h>

#include "dp_internal.h"

namespace dpk {
namespace {

constexpr int kMaxS = 64;
constexpr int kMaxK = 16;
constexpr int kHW = 1;      // warps per CTA (one: fine-grained occupancy for the register-heavy kernels)
constexpr int kChunk = 32;  // sequence symbols staged per refill

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

// Stage symbols [t0, t0 + kChunk) of the warp's sequences (0 past the end).
template <int NS>
__device__ __forceinline__ void stage_symbols(const HmmArgs& H, int64_t p0, const int* T, int t0, uint8_t (*xs)[kChunk],
                                              int lane) {
#pragma unroll
  for (int q = 0; q < NS; ++q) {
    const int64_t p = p0 + q;
    const int t = t0 + lane;
    xs[q][lane] = (p < H.n && t < T[q]) ? H.x_cat[H.x_off[p] + t] : 0;
  }
}

template <int NS>
__global__ void __launch_bounds__(kHW * 32) k_forward(HmmArgs H) {
  __shared__ __align__(16) float alpha[kHW][NS][kMaxS];
  __shared__ float Es[kMaxK][kMaxS];
  __shared__ uint8_t xs_all[kHW][NS][kChunk];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int S = H.S, K = H.K;
  for (int q = threadIdx.x; q < kMaxS * kMaxK; q += blockDim.x) {
    const int c = q / kMaxS, s = q % kMaxS;
    Es[c][s] = (s < S && c < K) ? H.E[s * K + c] : 0.f;
  }
  __syncthreads();
  const int64_t p0 = ((int64_t)blockIdx.x * kHW + warp) * NS;
  if (p0 >= H.n) return;
  uint8_t (*xs)[kChunk] = xs_all[warp];
  const int s0 = lane, s1 = lane + 32;
  float a0[kMaxS], a1[kMaxS];
#pragma unroll
  for (int q = 0; q < kMaxS; ++q) {
    a0[q] = (q < S && s0 < S) ? H.A[q * S + s0] : 0.f;
    a1[q] = (q < S && s1 < S) ? H.A[q * S + s1] : 0.f;
  }
  int T[NS];
  int Tmax = 0;
#pragma unroll
  for (int q = 0; q < NS; ++q) {
    T[q] = (p0 + q < H.n) ? (int)(H.x_off[p0 + q + 1] - H.x_off[p0 + q]) : 0;
    Tmax = max(Tmax, T[q]);
  }
  double ll[NS];
  float prod[NS];
  stage_symbols<NS>(H, p0, T, 0, xs, lane);
  __syncwarp();
  // i = 1: a(s) = pi_s e_s(x_1)
#pragma unroll
  for (int q = 0; q < NS; ++q) {
    ll[q] = 0.0;
    prod[q] = 1.f;
    const int c = xs[q][0];
    const float v0 = (s0 < S) ? H.pi[s0] * Es[c][s0] : 0.f;
    const float v1 = (s1 < S) ? H.pi[s1] * Es[c][s1] : 0.f;
    const float tot = warp_sum(v0 + v1);
    const float inv = 1.f / tot;
    prod[q] = tot;
    alpha[warp][q][s0] = v0 * inv;
    alpha[warp][q][s1] = v1 * inv;
  }
  __syncwarp();
  for (int i = 2; i <= Tmax; ++i) {
    if (((i - 1) & (kChunk - 1)) == 0) {
      __syncwarp();
      stage_symbols<NS>(H, p0, T, i - 1, xs, lane);
      __syncwarp();
    }
    float v0[NS], v1[NS];
#pragma unroll
    for (int q = 0; q < NS; ++q) {
      float acc0a = 0.f, acc0b = 0.f, acc1a = 0.f, acc1b = 0.f;
      const float4* al = reinterpret_cast<const float4*>(alpha[warp][q]);
#pragma unroll
      for (int q4 = 0; q4 < kMaxS / 4; ++q4) {
        const float4 v = al[q4];
        acc0a = fmaf(v.x, a0[4 * q4 + 0], acc0a);
        acc0b = fmaf(v.y, a0[4 * q4 + 1], acc0b);
        acc0a = fmaf(v.z, a0[4 * q4 + 2], acc0a);
        acc0b = fmaf(v.w, a0[4 * q4 + 3], acc0b);
        acc1a = fmaf(v.x, a1[4 * q4 + 0], acc1a);
        acc1b = fmaf(v.y, a1[4 * q4 + 1], acc1b);
        acc1a = fmaf(v.z, a1[4 * q4 + 2], acc1a);
        acc1b = fmaf(v.w, a1[4 * q4 + 3], acc1b);
      }
      const int c = xs[q][(i - 1) & (kChunk - 1)];
      v0[q] = (acc0a + acc0b) * Es[c][s0];
      v1[q] = (acc1a + acc1b) * Es[c][s1];
    }
    __syncwarp();
#pragma unroll
    for (int q = 0; q < NS; ++q) {
      if (i > T[q]) continue;  // warp-uniform
      const float tot = warp_sum(v0[q] + v1[q]);
      const float inv = 1.f / tot;
      alpha[warp][q][s0] = v0[q] * inv;
      alpha[warp][q][s1] = v1[q] * inv;
      prod[q] *= tot;
      if (!(prod[q] > 8.6736e-19f && prod[q] < 1.1529215e18f)) {  // outside [2^-60, 2^60]
        ll[q] += log((double)prod[q]);
        prod[q] = 1.f;
      }
    }
    __syncwarp();
  }
  if (lane == 0) {
#pragma unroll
    for (int q = 0; q < NS; ++q)
      if (p0 + q < H.n) H.ll_out[p0 + q] = T[q] == 0 ? 0.f : (float)(ll[q] + log((double)prod[q]));
  }
}

// One warp walks sequence p's back-pointers from its final state s (T >= 1), the path into
// o[0 .. T). The walk s_{i-1} = bp[i-1][s_i] is one dependent load per step; the warp stages the
// back-pointer rows it will need 32 at a time (row i-1 by lane T - i - 32c, one coalesced 2 KB
// read per chunk, the next chunk's loads in flight during the walk) in shared memory, lane 0
// walks the 32 steps there, and the warp writes the 32 states out with one coalesced store.
// fresh: the rows were just written by this kernel (L2 loads) rather than by an earlier one
// (streaming loads).
__device__ __forceinline__ void viterbi_walk(const HmmArgs& H, int64_t p, int T, int s, uint8_t* o,
                                             uint8_t (*rows)[32][kMaxS], uint8_t* ob, int lane, bool fresh) {
  const uint8_t* bp = H.bp + (p * H.max_len) * kMaxS;
  const int nch = (T + 31) / 32;
  // chunk c: lane t holds row r = T - 1 - 32 c - t (used at position i = r + 1), valid for r >= 1
  auto load = [&](int c, uint4* v) {
    const int r = T - 1 - 32 * c - lane;
    const uint4* src = reinterpret_cast<const uint4*>(bp + (int64_t)(r >= 1 ? r : 1) * kMaxS);
#pragma unroll
    for (int w = 0; w < kMaxS / 16; ++w)
      v[w] = r >= 1 ? (fresh ? __ldcg(src + w) : __ldcs(src + w)) : make_uint4(0, 0, 0, 0);
  };
  auto stash = [&](int buf, const uint4* v) {
    uint4* dst = reinterpret_cast<uint4*>(rows[buf][lane]);
#pragma unroll
    for (int w = 0; w < kMaxS / 16; ++w) dst[w] = v[w];
  };
  uint4 v[kMaxS / 16];
  load(0, v);
  stash(0, v);
  for (int c = 0; c < nch; ++c) {
    if (c + 1 < nch) load(c + 1, v);   // in flight during the walk
    __syncwarp();
    if (lane == 0) {
      const uint8_t* R = &rows[c & 1][0][0];
      for (int t = 0; t < 32; ++t) {
        const int i = T - 32 * c - t;   // position
        if (i < 1) break;
        ob[t] = (uint8_t)s;
        if (i >= 2) s = R[t * kMaxS + s];
      }
    }
    __syncwarp();
    const int i = T - 32 * c - lane;
    if (i >= 1) o[i - 1] = ob[lane];
    if (c + 1 < nch) stash((c + 1) & 1, v);
  }
  __syncwarp();
}

constexpr int kNegKey = -(1 << 30);
constexpr int kRenorm = 32;

template <int NS>
__global__ void __launch_bounds__(kHW * 32) k_viterbi(HmmArgs H) {
  __shared__ __align__(16) int key[kHW][NS][kMaxS];
  __shared__ int Es[kMaxK][kMaxS];
  __shared__ uint8_t xs_all[kHW][NS][kChunk];
  __shared__ __align__(16) uint8_t walk_rows[kHW][2][32][kMaxS];  // the fused walk's staged rows
  __shared__ uint8_t walk_ob[kHW][32];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int S = H.S, K = H.K;
  for (int q = threadIdx.x; q < kMaxS * kMaxK; q += blockDim.x) {
    const int c = q / kMaxS, s = q % kMaxS;
    Es[c][s] = (s < S && c < K) ? H.lE[s * K + c] : 0;
  }
  __syncthreads();
  const int64_t p0 = ((int64_t)blockIdx.x * kHW + warp) * NS;
  if (p0 >= H.n) return;
  uint8_t (*xs)[kChunk] = xs_all[warp];
  const int s0 = lane, s1 = lane + 32;
  const bool ok0 = s0 < S, ok1 = s1 < S;
  int la0[kMaxS], la1[kMaxS];  // transition scores x 64 (key units)
#pragma unroll
  for (int q = 0; q < kMaxS; ++q) {
    la0[q] = (q < S && ok0) ? H.lA[q * S + s0] * 64 : 0;
    la1[q] = (q < S && ok1) ? H.lA[q * S + s1] * 64 : 0;
  }
  int T[NS];
  int Tmax = 0;
#pragma unroll
  for (int q = 0; q < NS; ++q) {
    T[q] = (p0 + q < H.n) ? (int)(H.x_off[p0 + q + 1] - H.x_off[p0 + q]) : 0;
    Tmax = max(Tmax, T[q]);
  }
  stage_symbols<NS>(H, p0, T, 0, xs, lane);
  __syncwarp();
  int V0[NS], V1[NS];
  int64_t off[NS];
#pragma unroll
  for (int q = 0; q < NS; ++q) {
    const int c = xs[q][0];
    V0[q] = ok0 ? H.lpi[s0] + Es[c][s0] : kNegKey;
    V1[q] = ok1 ? H.lpi[s1] + Es[c][s1] : kNegKey;
    const int m = warp_max(max(V0[q], V1[q]));
    off[q] = m;
    V0[q] -= m; V1[q] -= m;
    key[warp][q][s0] = ok0 ? V0[q] * 64 + (63 - s0) : kNegKey;
    key[warp][q][s1] = ok1 ? V1[q] * 64 + (63 - s1) : kNegKey;
  }
  __syncwarp();
  for (int i = 2; i <= Tmax; ++i) {
    if (((i - 1) & (kChunk - 1)) == 0) {
      __syncwarp();
      stage_symbols<NS>(H, p0, T, i - 1, xs, lane);
      __syncwarp();
    }
    int k0[NS], k1[NS];
#pragma unroll
    for (int q = 0; q < NS; ++q) {
      int b0a = INT32_MIN, b0b = INT32_MIN, b1a = INT32_MIN, b1b = INT32_MIN;
      const int4* kv = reinterpret_cast<const int4*>(key[warp][q]);
#pragma unroll
      for (int q4 = 0; q4 < kMaxS / 4; ++q4) {
        const int4 v = kv[q4];
        b0a = __viaddmax_s32(v.x, la0[4 * q4 + 0], b0a);
        b0b = __viaddmax_s32(v.y, la0[4 * q4 + 1], b0b);
        b0a = __viaddmax_s32(v.z, la0[4 * q4 + 2], b0a);
        b0b = __viaddmax_s32(v.w, la0[4 * q4 + 3], b0b);
        b1a = __viaddmax_s32(v.x, la1[4 * q4 + 0], b1a);
        b1b = __viaddmax_s32(v.y, la1[4 * q4 + 1], b1b);
        b1a = __viaddmax_s32(v.z, la1[4 * q4 + 2], b1a);
        b1b = __viaddmax_s32(v.w, la1[4 * q4 + 3], b1b);
      }
      k0[q] = max(b0a, b0b);
      k1[q] = max(b1a, b1b);
    }
    __syncwarp();
#pragma unroll
    for (int q = 0; q < NS; ++q) {
      if (i > T[q]) continue;  // warp-uniform
      const int c = xs[q][(i - 1) & (kChunk - 1)];
      // key = V(p)*64 + (63-p) + lA*64  ->  floor(key / 64) = V(p) + lA, low 6 bits = 63 - argmax
      V0[q] = ok0 ? (k0[q] >> 6) + Es[c][s0] : kNegKey;
      V1[q] = ok1 ? (k1[q] >> 6) + Es[c][s1] : kNegKey;
      if (H.bp) {
        uint8_t* bp = H.bp + ((p0 + q) * H.max_len + (i - 1)) * kMaxS;
        if (ok0) bp[s0] = (uint8_t)(63 - (k0[q] & 63));
        if (ok1) bp[s1] = (uint8_t)(63 - (k1[q] & 63));
      }
      if ((i & (kRenorm - 1)) == 0) {
        const int m = warp_max(max(V0[q], V1[q]));
        off[q] += m;
        V0[q] -= m; V1[q] -= m;
      }
      key[warp][q][s0] = ok0 ? V0[q] * 64 + (63 - s0) : kNegKey;
      key[warp][q][s1] = ok1 ? V1[q] * 64 + (63 - s1) : kNegKey;
    }
    __syncwarp();
  }
  // best final state: max V, lowest index on ties -> max of V*64 + (63 - s)
#pragma unroll
  for (int q = 0; q < NS; ++q) {
    const int fk = warp_max(max(key[warp][q][s0], key[warp][q][s1]));
    if (lane == 0 && p0 + q < H.n) {
      if (T[q] == 0) {
        H.vit_out[p0 + q] = 0;
        if (H.final_state) H.final_state[p0 + q] = -1;
      } else {
        H.vit_out[p0 + q] = (int32_t)(off[q] + (fk >> 6));
        if (H.final_state) H.final_state[p0 + q] = 63 - (fk & 63);
      }
    }
    // the walk right behind the sweep: this warp's back-pointers were just written (L2-resident),
    // and other warps' sweeps keep the SM busy while it waits on them
    if (H.path && p0 + q < H.n && T[q] > 0) {
      __syncwarp();  // the final state and every back-pointer row of this warp are written
      viterbi_walk(H, p0 + q, T[q], 63 - (fk & 63), H.path + (p0 + q) * H.max_len, walk_rows[warp], walk_ob[warp],
                   lane, true);
    }
  }
}

// Viterbi traceback (dp_traceback): the paths were walked by k_viterbi right behind the sweep
// (viterbi_walk); this copies rows [first, first + count) into the caller's layout, one warp per
// row. k_viterbi_tb (the walk as a kernel of its own) serves plans whose solve did not walk.
constexpr int kTbW = 4;  // warps per CTA

__global__ void __launch_bounds__(kTbW * 32) k_viterbi_copy(HmmArgs H, int64_t first, int64_t count, uint8_t* out,
                                                             int64_t stride, int32_t* out_len) {
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  for (int64_t q = (int64_t)blockIdx.x * kTbW + warp; q < count; q += (int64_t)gridDim.x * kTbW) {
    const int64_t p = first + q;
    const int T = (int)(H.x_off[p + 1] - H.x_off[p]);
    if (T > stride) {
      if (lane == 0) out_len[q] = -1;
      continue;
    }
    const uint8_t* src = H.path + p * H.max_len;
    uint8_t* o = out + q * stride;
    for (int i = lane; i < T; i += 32) o[i] = src[i];
    if (lane == 0) out_len[q] = T;
  }
}

__global__ void __launch_bounds__(kTbW * 32) k_viterbi_tb(HmmArgs H, int64_t first, int64_t count, uint8_t* out,
                                                           int64_t stride, int32_t* out_len) {
  __shared__ __align__(16) uint8_t rows[kTbW][2][32][kMaxS];
  __shared__ uint8_t ob[kTbW][32];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  for (int64_t q = (int64_t)blockIdx.x * kTbW + warp; q < count; q += (int64_t)gridDim.x * kTbW) {
    const int64_t p = first + q;
    const int T = (int)(H.x_off[p + 1] - H.x_off[p]);
    if (T > stride) {
      if (lane == 0) out_len[q] = -1;
      continue;
    }
    if (T > 0) viterbi_walk(H, p, T, H.final_state[p], out + q * stride, rows[warp], ob[warp], lane, false);
    if (lane == 0) out_len[q] = T;
  }
}

int sms_of_current() {
  int dev = 0, v = 0;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&v, cudaDevAttrMultiProcessorCount, dev);
  return v > 0 ? v : 148;
}

template <int NS>
void* fwd_ptr(bool viterbi) { return viterbi ? (void*)k_viterbi<NS> : (void*)k_forward<NS>; }

// Sequences per warp: minimise (waves of resident warps) x (NS + latency term): the per-warp
// time grows with NS plus (forward) a latency term that NS independent sequences share;
// ties go to the smaller NS.
int pick_ns(int64_t n, bool viterbi, void** kern, int ns_override) {
  void* ks[8] = {fwd_ptr<1>(viterbi), fwd_ptr<2>(viterbi), fwd_ptr<3>(viterbi), fwd_ptr<4>(viterbi),
                 fwd_ptr<5>(viterbi), fwd_ptr<6>(viterbi), fwd_ptr<7>(viterbi), fwd_ptr<8>(viterbi)};
  const int sms = sms_of_current();
  int best = 1;
  int64_t best_cost = INT64_MAX;
  for (int ns = 1; ns <= 8; ++ns) {
    int per_sm = 0;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, ks[ns - 1], kHW * 32, 0) != cudaSuccess || per_sm < 1)
      continue;
    const int64_t warps = (n + ns - 1) / ns;
    const int64_t wave = (int64_t)sms * per_sm * kHW;
    // Viterbi: measured (10k x 1000, S = 64) NS = 1 / 2 / 3 / 4 -> 2.99 / 3.57 / 3.86 / 3.95 ms, so no
    // latency term; the SIMT forward keeps it
    const int64_t cost = ((warps + wave - 1) / wave) * (ns + (viterbi ? 0 : 2));
    if (cost < best_cost) { best_cost = cost; best = ns; }
  }
  if (ns_override > 0) best = std::max(1, std::min(8, ns_override));  // diagnostic (DP_HMM_NS)
  *kern = ks[best - 1];
  return best;
}

}  // namespace

cudaError_t hmm_forward(const HmmArgs& H, cudaStream_t s, int64_t* launches) {
  if (H.n == 0) return cudaSuccess;
  void* kern = nullptr;
  const int ns = pick_ns(H.n, false, &kern, H.ns_override);
  const int64_t warps = (H.n + ns - 1) / ns;
  HmmArgs h2 = H;
  void* args[1] = {&h2};
  ++*launches;
  return cudaLaunchKernel(kern, dim3((unsigned)((warps + kHW - 1) / kHW)), dim3(kHW * 32), args, 0, s);
}

cudaError_t hmm_viterbi(const HmmArgs& H, cudaStream_t s, int64_t* launches) {
  if (H.n == 0) return cudaSuccess;
  void* kern = nullptr;
  const int ns = pick_ns(H.n, true, &kern, H.ns_override);
  const int64_t warps = (H.n + ns - 1) / ns;
  HmmArgs h2 = H;
  void* args[1] = {&h2};
  ++*launches;
  return cudaLaunchKernel(kern, dim3((unsigned)((warps + kHW - 1) / kHW)), dim3(kHW * 32), args, 0, s);
}

cudaError_t hmm_viterbi_traceback(const HmmArgs& H, int64_t first, int64_t count, uint8_t* out, int64_t stride,
                                  int32_t* out_len, cudaStream_t s, int64_t* launches) {
  if (count == 0) return cudaSuccess;
  const int64_t grid = std::min<int64_t>((count + kTbW - 1) / kTbW, (int64_t)sms_of_current() * 12);
  ++*launches;
  if (H.path) k_viterbi_copy<<<(unsigned)grid, kTbW * 32, 0, s>>>(H, first, count, out, stride, out_len);
  else k_viterbi_tb<<<(unsigned)grid, kTbW * 32, 0, s>>>(H, first, count, out, stride, out_len);
  return cudaGetLastError();
}

}  // namespace dpk
