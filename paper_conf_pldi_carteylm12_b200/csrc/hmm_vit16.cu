// Viterbi in s16x2: two sequences per warp register (DESIGN.md §3.3 "k_viterbi16").
//
// The recurrence is the max-variant of Fig.11a (R-VIT): V_i(r) =
// max_p (V_{i-1}(p) + lA(p, r)) + lE(r, x_i) in int32 milli-bits. k_viterbi (hmm.cu) runs it on
// int32 keys V * 64 + (63 - p), one VIADDMNMX per (p, r) carrying both the max and the argmax.
// Here the max runs on packed 16-bit halves — sequence a in the low half, b in the high half of
// every register — so one VIADDMNMX.S16x2 does a (p, r) term for two sequences, and the argmax is
// recovered along the optimal path only, by the walk at the end (it needs one row per position).
//
// Exactness in 16 bits (rows relative to their maximum, per column / per symbol offsets):
//   a'(p, r) = lA(p, r) - c_r with c_r = max_p lA(p, r), A' = max_r (max_p - min_p) of lA(., r);
//   e'(r, x) = lE(r, x) + c_r, e''(r, x) = e'(r, x) - emax(x) with emax(x) = max_r e'(r, x);
//   the stored row is rel(p) = max(V(p) - off, -C) with off the row's true maximum, C = 32768 - A'.
// With C >= A' + 1 (A' <= 16383, checked on the host at plan creation, else k_viterbi) a state
// whose true rel is below -C is strictly worse, for every r, than the row's maximum state p*
// (rel(p) + a'(p, r) < -C <= -A' - 1 < a'(p*, r)), so clamping it changes no maximum, no argmax and
// no tie. Every sum stays in range: rel + a' >= -C - A' = -32768; acc(r) = max_p (rel + a') >=
// a'(p*, r) >= -A'; new(r) = acc(r) + e'' >= -A' - E'' (saturating add when that can pass -32768:
// a saturated value is still <= -C after the shift, because the row maximum M >= -A' — the state
// with e'' = 0 keeps acc >= -A'). V_i = new + off_{i-1} + emax(x_i), off_i = off_{i-1} + emax(x_i) + M_i.
#include <algorithm>
#include <climits>
#include <cstdint>
#include <cstdlib>
#include <cuda_runtime.h>

#include "dp_internal.h"

namespace dpk {
namespace {

constexpr int kS = 64;
constexpr int kK = 16;
constexpr int kCh = 32;    // symbols staged per refill
constexpr int kWalkD = 8;  // rows prefetched per walk block

struct V16Smem {
  uint32_t row[2][kS];    // the pair's previous row, packed (a | b << 16); double-buffered
  uint32_t E2[kK][kS];    // e''(r, x), the same value in both halves
  uint32_t at2[kS][33];   // walk: a'(l, s) | a'(l + 32, s) << 16 at [s][l] (33: conflict-free fill)
  int emax[kK];
  uint8_t xs[2][kCh];
};

__device__ __forceinline__ uint32_t pk(int lo, int hi) { return (uint32_t)(lo & 0xffff) | ((uint32_t)hi << 16); }
// an opaque copy: keeps the compiler from holding a packed constant as its two halves and
// re-packing it every step (it does that to the transition registers otherwise)
__device__ __forceinline__ uint32_t opaque(uint32_t x) {
  uint32_t y;
  asm volatile("mov.b32 %0, %1;" : "=r"(y) : "r"(x));
  return y;
}
__device__ __forceinline__ int lo16(uint32_t x) { return (int)(int16_t)(x & 0xffffu); }
__device__ __forceinline__ int hi16(uint32_t x) { return (int)x >> 16; }

// Walk of one sequence (NH = 1: the half `hi` of the rows) or of both (NH = 2, equal lengths T):
// step j moves from position i = T - j to i - 1 with the row of position i - 1 (stored at index
// i - 2, lane l holding states l and l + 32). Keys (v + a') * 64 + (63 - p): one REDUX per step
// gives the maximum and its lowest index; inactive states (p >= S) hold -C with a' = 0 and never
// reach the maximum (see the header). The rows are prefetched kWalkD steps ahead; lane t keeps
// the state of step 32 c + t and the warp writes 32 path bytes at a time.
template <int NH>
__device__ __forceinline__ void walk16(const uint2* rws, int T, int sA, int sB, bool hi, uint8_t* oA, uint8_t* oB,
                                       const uint32_t (*at2)[33], int lane) {
  const int J = T - 1;  // steps that move
  const int key0 = 63 - lane, key1 = 31 - lane;
  uint32_t keepA = 0, keepB = 0;
  auto ld = [&](int j) { return j < J ? __ldcg(rws + (int64_t)(T - j - 2) * 32 + lane) : make_uint2(0, 0); };
  auto move = [&](int s, uint2 v, bool h) {
    const uint32_t a2 = at2[s][lane];
    const int v0 = h ? hi16(v.x) : lo16(v.x), v1 = h ? hi16(v.y) : lo16(v.y);
    const int k = max((v0 + lo16(a2)) * 64 + key0, (v1 + hi16(a2)) * 64 + key1);
    return (~__reduce_max_sync(0xffffffffu, k)) & 63;  // 63 - (key & 63)
  };
  auto flush = [&](int j) {
    const int jj = (j & ~31) + lane;
    if (jj <= j) {
      oA[T - 1 - jj] = (uint8_t)keepA;
      if (NH == 2) oB[T - 1 - jj] = (uint8_t)keepB;
    }
  };
  uint2 cur[kWalkD], nxt[kWalkD];
#pragma unroll
  for (int k = 0; k < kWalkD; ++k) cur[k] = ld(k);
  for (int jb = 0; jb < J; jb += kWalkD) {
#pragma unroll
    for (int k = 0; k < kWalkD; ++k) nxt[k] = ld(jb + kWalkD + k);
#pragma unroll
    for (int k = 0; k < kWalkD; ++k) {
      const int j = jb + k;
      if (j >= J) break;
      if (lane == (j & 31)) keepA = sA, keepB = sB;
      sA = move(sA, cur[k], NH == 2 ? false : hi);
      if (NH == 2) sB = move(sB, cur[k], true);
      if ((j & 31) == 31) flush(j);
    }
#pragma unroll
    for (int k = 0; k < kWalkD; ++k) cur[k] = nxt[k];
  }
  if (lane == (J & 31)) keepA = sA, keepB = sB;  // position 1
  flush(J);
}

// FULL: S == 64, every lane's two states exist (no per-step masking)
template <bool SAT, bool FULL>
__global__ void __launch_bounds__(32) k_viterbi16(HmmArgs H) {
  __shared__ __align__(16) V16Smem sm;
  const int lane = threadIdx.x;
  const int S = FULL ? kS : H.S, K = H.K;
  const int64_t pa = 2 * (int64_t)blockIdx.x, pb = pa + 1;
  const int s0 = lane, s1 = lane + 32;
  const bool ok0 = FULL || s0 < S, ok1 = FULL || s1 < S;
  const int Ta = pa < H.n ? (int)(H.x_off[pa + 1] - H.x_off[pa]) : 0;
  const int Tb = pb < H.n ? (int)(H.x_off[pb + 1] - H.x_off[pb]) : 0;
  const int Tmax = max(Ta, Tb);
  const int C = H.v16_C;
  const uint32_t Cpk = pk(-C, -C);

  // the owned columns r = s0, s1 of a', both halves alike
  int c0 = 0, c1 = 0;
  if (ok0) {
    c0 = INT_MIN;
    for (int q = 0; q < S; ++q) c0 = max(c0, H.lA[q * S + s0]);
  }
  if (ok1) {
    c1 = INT_MIN;
    for (int q = 0; q < S; ++q) c1 = max(c1, H.lA[q * S + s1]);
  }
  uint32_t la0[kS], la1[kS];
#pragma unroll
  for (int q = 0; q < kS; ++q) {
    const int v0 = (q < S && ok0) ? H.lA[q * S + s0] - c0 : 0;
    const int v1 = (q < S && ok1) ? H.lA[q * S + s1] - c1 : 0;
    la0[q] = opaque(pk(v0, v0));
    la1[q] = opaque(pk(v1, v1));
  }
  // emission tables: emax(x) = max_r e'(r, x), E2 = e'' = e' - emax
  for (int x = 0; x < kK; ++x) {
    const int e0 = (x < K && ok0) ? H.lE[s0 * K + x] + c0 : INT_MIN;
    const int e1 = (x < K && ok1) ? H.lE[s1 * K + x] + c1 : INT_MIN;
    const int em = __reduce_max_sync(0xffffffffu, max(e0, e1));
    const int d0 = ok0 && x < K ? e0 - em : 0, d1 = ok1 && x < K ? e1 - em : 0;
    sm.E2[x][s0] = pk(d0, d0);
    sm.E2[x][s1] = pk(d1, d1);
    if (lane == 0) sm.emax[x] = x < K ? em : 0;
  }
  if (H.path) {
#pragma unroll
    for (int l = 0; l < 32; ++l) {
      sm.at2[s0][l] = pk(lo16(la0[l]), lo16(la0[l + 32]));
      sm.at2[s1][l] = pk(lo16(la1[l]), lo16(la1[l + 32]));
    }
  }
  auto stage = [&](int t0) {
    const int t = t0 + lane;
    sm.xs[0][lane] = t < Ta ? H.x_cat[H.x_off[pa] + t] : 0;
    sm.xs[1][lane] = t < Tb ? H.x_cat[H.x_off[pb] + t] : 0;
  };
  stage(0);
  __syncwarp();

  int64_t offa = 0, offb = 0;
  int fa = -1, fb = -1;  // final states
  int64_t va = 0, vb = 0;  // final scores (the offsets at T: the row maximum is 0 there)
  uint32_t* rows = H.rows16 ? H.rows16 + (int64_t)blockIdx.x * H.max_len * kS : nullptr;
  // final state of a row (max rel = 0): the lowest such index
  auto final_state = [&](uint32_t r0, uint32_t r1, bool hi) {
    const int v0 = hi ? hi16(r0) : lo16(r0), v1 = hi ? hi16(r1) : lo16(r1);
    const int cand = (ok0 && v0 == 0) ? s0 : (ok1 && v1 == 0) ? s1 : kS;
    return (int)__reduce_min_sync(0xffffffffu, (unsigned)cand);
  };
  if (Tmax > 0) {  // i = 1: V_1(s) = lpi(s) + lE(s, x_1), exact in int32, then shifted and clamped
    const int ca = sm.xs[0][0], cb = sm.xs[1][0];
    constexpr int kNeg = -(1 << 30);
    const int va0 = ok0 ? H.lpi[s0] + H.lE[s0 * K + ca] : kNeg, va1 = ok1 ? H.lpi[s1] + H.lE[s1 * K + ca] : kNeg;
    const int vb0 = ok0 ? H.lpi[s0] + H.lE[s0 * K + cb] : kNeg, vb1 = ok1 ? H.lpi[s1] + H.lE[s1 * K + cb] : kNeg;
    const int Ma = __reduce_max_sync(0xffffffffu, max(va0, va1));
    const int Mb = __reduce_max_sync(0xffffffffu, max(vb0, vb1));
    offa = Ma;
    offb = Mb;
    const uint32_t r0 = pk(max(va0 - Ma, -C), max(vb0 - Mb, -C));
    const uint32_t r1 = pk(max(va1 - Ma, -C), max(vb1 - Mb, -C));
    sm.row[1][s0] = r0;
    sm.row[1][s1] = r1;
    if (rows && Tmax > 1) reinterpret_cast<uint2*>(rows)[lane] = make_uint2(r0, r1);
    if (Ta == 1) fa = final_state(r0, r1, false), va = offa;
    if (Tb == 1) fb = final_state(r0, r1, true), vb = offb;
  }
  __syncwarp();
  const int Tmin = min(Ta, Tb);
  for (int i = 2; i <= Tmax; ++i) {
    if (((i - 1) & (kCh - 1)) == 0) {
      __syncwarp();
      stage(i - 1);
      __syncwarp();
    }
    const uint4* rv = reinterpret_cast<const uint4*>(sm.row[(i - 1) & 1]);
    uint32_t b0a = 0x80008000u, b0b = 0x80008000u, b1a = 0x80008000u, b1b = 0x80008000u;
#pragma unroll
    for (int q4 = 0; q4 < kS / 4; ++q4) {
      const uint4 v = rv[q4];
      b0a = __viaddmax_s16x2(v.x, la0[4 * q4 + 0], b0a);
      b0b = __viaddmax_s16x2(v.y, la0[4 * q4 + 1], b0b);
      b0a = __viaddmax_s16x2(v.z, la0[4 * q4 + 2], b0a);
      b0b = __viaddmax_s16x2(v.w, la0[4 * q4 + 3], b0b);
      b1a = __viaddmax_s16x2(v.x, la1[4 * q4 + 0], b1a);
      b1b = __viaddmax_s16x2(v.y, la1[4 * q4 + 1], b1b);
      b1a = __viaddmax_s16x2(v.z, la1[4 * q4 + 2], b1a);
      b1b = __viaddmax_s16x2(v.w, la1[4 * q4 + 3], b1b);
    }
    const int ca = sm.xs[0][(i - 1) & (kCh - 1)], cb = sm.xs[1][(i - 1) & (kCh - 1)];
    const uint32_t e0 = __byte_perm(sm.E2[ca][s0], sm.E2[cb][s0], 0x7610);
    const uint32_t e1 = __byte_perm(sm.E2[ca][s1], sm.E2[cb][s1], 0x7610);
    const uint32_t acc0 = __vmaxs2(b0a, b0b), acc1 = __vmaxs2(b1a, b1b);
    uint32_t n0 = SAT ? __vaddss2(acc0, e0) : __vadd2(acc0, e0);
    uint32_t n1 = SAT ? __vaddss2(acc1, e1) : __vadd2(acc1, e1);
    if (!ok0) n0 = 0x80008000u;
    if (!ok1) n1 = 0x80008000u;
    const uint32_t m = __vmaxs2(n0, n1);
    // the halves' maxima, shifted up 16: their negations' high halves are -M, packed by one PRMT
    const int Ra = __reduce_max_sync(0xffffffffu, (int)(m << 16));
    const int Rb = __reduce_max_sync(0xffffffffu, (int)(m & 0xffff0000u));
    const int Ma = Ra >> 16, Mb = Rb >> 16;
    const uint32_t negM = __byte_perm(0u - (uint32_t)Ra, 0u - (uint32_t)Rb, 0x7632);
    const uint32_t r0 = __viaddmax_s16x2(n0, negM, Cpk);
    const uint32_t r1 = __viaddmax_s16x2(n1, negM, Cpk);
    offa += sm.emax[ca] + Ma;
    offb += sm.emax[cb] + Mb;
    sm.row[i & 1][s0] = r0;
    sm.row[i & 1][s1] = r1;
    if (rows && i < Tmax)  // row of position i, read by the walk at position i + 1
      reinterpret_cast<uint2*>(rows + (int64_t)(i - 1) * kS)[lane] = make_uint2(r0, r1);
    if (i >= Tmin) {  // warp-uniform; only the last steps of the shorter sequence
      if (i == Ta) fa = final_state(r0, r1, false), va = offa;
      if (i == Tb) fb = final_state(r0, r1, true), vb = offb;
    }
    __syncwarp();
  }
  if (lane == 0) {
    if (pa < H.n) {
      H.vit_out[pa] = Ta == 0 ? 0 : (int32_t)va;
      if (H.final_state) H.final_state[pa] = Ta == 0 ? -1 : fa;
    }
    if (pb < H.n) {
      H.vit_out[pb] = Tb == 0 ? 0 : (int32_t)vb;
      if (H.final_state) H.final_state[pb] = Tb == 0 ? -1 : fb;
    }
  }
  if (!H.path || Tmax == 0) return;

  // The walks: s_{i-1} = argmax_p rel_{i-1}(p) + a'(p, s_i), lowest p on ties; both sequences
  // in one loop when their lengths agree (they share the rows), else one after the other.
  const uint2* rws = reinterpret_cast<const uint2*>(H.rows16 + (int64_t)blockIdx.x * H.max_len * kS);
  uint8_t* oa = H.path + pa * H.max_len;
  uint8_t* ob = H.path + pb * H.max_len;
  if (Ta == Tb) {
    walk16<2>(rws, Ta, fa, fb, false, oa, ob, sm.at2, lane);
  } else {
    if (Ta > 0) walk16<1>(rws, Ta, fa, 0, false, oa, nullptr, sm.at2, lane);
    if (Tb > 0) walk16<1>(rws, Tb, fb, 0, true, ob, nullptr, sm.at2, lane);
  }
}

}  // namespace

// Host-side guard (plan creation): the 16-bit formulation is exact when A' <= 16383; the
// saturating add is needed when A' + E'' can pass 32768. Returns C = 32768 - A' (> 0) or 0.
int vit16_clamp(const int32_t* lA, const int32_t* lE, int S, int K, int* sat) {
  int64_t Ap = 0;
  int64_t c[kS];
  for (int r = 0; r < S; ++r) {
    int64_t mx = INT64_MIN, mn = INT64_MAX;
    for (int p = 0; p < S; ++p) {
      mx = std::max<int64_t>(mx, lA[p * S + r]);
      mn = std::min<int64_t>(mn, lA[p * S + r]);
    }
    c[r] = mx;
    Ap = std::max<int64_t>(Ap, mx - mn);
  }
  if (Ap > 16383) return 0;
  int64_t Epp = 0;
  for (int x = 0; x < K; ++x) {
    int64_t em = INT64_MIN, en = INT64_MAX;
    for (int r = 0; r < S; ++r) {
      em = std::max<int64_t>(em, lE[r * K + x] + c[r]);
      en = std::min<int64_t>(en, lE[r * K + x] + c[r]);
    }
    Epp = std::max<int64_t>(Epp, em - en);
  }
  *sat = (Ap + Epp > 32768) ? 1 : 0;
  return (int)(32768 - Ap);
}

cudaError_t hmm_viterbi16(const HmmArgs& H, cudaStream_t s, int64_t* launches) {
  if (H.n == 0) return cudaSuccess;
  HmmArgs h2 = H;
  void* args[1] = {&h2};
  ++*launches;
  const unsigned grid = (unsigned)((H.n + 1) / 2);
  void* kern = H.S == kS ? (H.v16_sat ? (void*)k_viterbi16<true, true> : (void*)k_viterbi16<false, true>)
                         : (H.v16_sat ? (void*)k_viterbi16<true, false> : (void*)k_viterbi16<false, false>);
  return cudaLaunchKernel(kern, dim3(grid), dim3(32),
                          args, 0, s);
}

}  // namespace dpk
