// Profile-HMM forward (§6.3): a database search, one
// profile of L match positions against a batch of sequences.
//
// Written as the paper's generic HMM (§5.2) the profile's silent delete states read the SAME
// sequence index, so with the "any state" reading of `transitionsto` (L466–L472) the dependency
// families are cyclic and no schedule exists. With the states in position-major order — the
// ordering the paper's Further Work says decides the schedules (L590–L592) — the forward is three
// mutually recursive tables over (j = position, i = sequence index) with uniform descents
//   M(j,i) = eM_j(x_i) [M(j-1,i-1) t^j_MM + I(j-1,i-1) t^j_IM + D(j-1,i-1) t^j_DM]     (-1,-1)
//   I(j,i) = eI_j(x_i) [M(j,i-1)   t^j_MI + I(j,i-1)   t^j_II + D(j,i-1)   t^j_DI]     ( 0,-1)
//   D(j,i) =            M(j-1,i)   t^j_MD + I(j-1,i)   t^j_ID + D(j-1,i)   t^j_DD      (-1, 0)
// (t^j_XY = the transition from X_{j-1} (M, D) or X_j (I) to Y; M_0 = begin, M_{L+1} = end),
// i.e. the edit-distance families: schedule (1,1), the anti-diagonal wavefront of k_align /
// k_sw16 (window 2, §4.8). P(x) = M(L,T) t_ME + I(L,T) t_IE + D(L,T) t_DE.
//
// Layout: one warp per sequence; lane l owns rows j = 1 + 256 st + 8 l + r (r < 8) of strip st and
// works on column i = k - l at step k; the row above travels down the warp by __shfl_up_sync (the
// new column) and the value shuffled one step earlier (the diagonal). Row 0 (I_0, begin) is a
// register of lane 0; between strips the last row goes through shared memory, per column.
// Transition coefficients live in registers (9 per row), the emission pairs (eM_j(c), eI_j(c)) per
// residue c in a shared table laid out per lane (one LDS.128 per two rows, conflict-free; see the
// kernel), dead residue K -> 0.
//
// Range: probabilities underflow fp32 after ~100 columns, so values are kept in scaled linear
// space (the paper lets the framework pick the probability representation, §3.2) with
// one power-of-two exponent per lane: stored = true * 2^-s. The exponent travels with the
// boundary row (an exact power-of-two rescale of the incoming values), a lane renormalises to
// its own maximum every 4 steps, and a lane whose values are negligible next to its input
// adopts the input's exponent (an all-zero lane takes the first nonzero input's). log P = log(stored) + s ln 2.
#include <cstdint>
#include <cuda_runtime.h>

#include "dp_internal.h"

namespace dpk {
namespace {

constexpr int kR = 8;             // rows per lane
constexpr int kStripRows = 32 * kR;
constexpr int kPW = 8;            // warps (sequences) per CTA

struct Tr9 {
  float mm, im, dm;   // into M_j from M_{j-1}, I_{j-1}, D_{j-1}
  float mi, ii, di;   // into I_j from M_j, I_j, D_j
  float md, id, dd;   // into D_j from M_{j-1}, I_{j-1}, D_{j-1}
};

// 2^d as a float for d in [-126, 127]; 0 below (the input is negligible at this scale)
__device__ __forceinline__ float exp2i(int d) {
  d = max(d, -127);
  d = min(d, 127);
  return d == -127 ? 0.0f : __int_as_float((d + 127) << 23);
}

__global__ void __launch_bounds__(kPW * 32, 2) k_phmm_forward(PhmmArgs A) {
  extern __shared__ __align__(16) uint8_t smem[];
  const int L = A.L, K = A.K;
  // Emission table, bank-conflict free: per residue c (c = K: the dead residue) S = 128 x strips
  // 16-byte chunks; the chunk of lane l's rows j0 + 2k, j0 + 2k + 1 (j0 = 1 + 256 st + 8 l) sits at
  // 128 st + 32 k + l and holds (eM, eI) of both rows. A step's four loads per lane (k = 0..3) then
  // put the 8 lanes of a quarter-warp on 8 distinct bank quads whatever residues their columns
  // hold (the row-major table had lanes 2 apart on the same quad: 73 % of the wavefronts were
  // conflicts). Row 0 (I_0's emissions) is a separate [K + 1] table.
  const int S = A.rows_tab;  // chunks per residue (128 x strips)
  float4* em = reinterpret_cast<float4*>(smem);
  float* ei0t = reinterpret_cast<float*>(em + (size_t)(K + 1) * S);
  for (int q = threadIdx.x; q < (K + 1) * S; q += blockDim.x) {
    const int c = q / S, h = q - c * S;
    const int st = h >> 7, k = (h >> 5) & 3, l = h & 31;
    const int r0 = 1 + 256 * st + 8 * l + 2 * k;
    float4 v = make_float4(0.f, 0.f, 0.f, 0.f);
    if (c < K && r0 <= L) { v.x = A.emit_m[r0 * K + c]; v.y = A.emit_i[r0 * K + c]; }
    if (c < K && r0 + 1 <= L) { v.z = A.emit_m[(r0 + 1) * K + c]; v.w = A.emit_i[(r0 + 1) * K + c]; }
    em[q] = v;
  }
  for (int c = threadIdx.x; c <= K; c += blockDim.x) ei0t[c] = c < K ? A.emit_i[c] : 0.f;
  __syncthreads();
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int64_t p = (int64_t)blockIdx.x * kPW + warp;
  if (p >= A.n) return;
  const uint8_t* x = A.x_cat + A.x_off[p];
  const int T = (int)(A.x_off[p + 1] - A.x_off[p]);
  const int strips = (L + kStripRows - 1) / kStripRows;
  // strip boundary (last row of the strip above, per column): M, I, D and the lane exponent
  float4* bnd = reinterpret_cast<float4*>(smem + (size_t)(K + 1) * S * sizeof(float4) + 128 * sizeof(float)) +
                (size_t)warp * (A.max_len + 1);
  const int jL = L;  // the last row: its owner lane captures P at column T
  float out_val = 0.f;
  int out_exp = 0;
  bool have_out = false;

  for (int st = 0; st < strips; ++st) {
    const int j0 = 1 + st * kStripRows + lane * kR;  // my first row
    Tr9 t[kR];
#pragma unroll
    for (int r = 0; r < kR; ++r) {
      const int j = j0 + r;
      if (j <= L) {
        const float* a = A.trans + (j - 1) * 9;  // from position j-1
        const float* b = A.trans + j * 9;        // from position j (into I_j)
        t[r] = {a[0], a[3], a[6], b[1], b[4], b[7], a[2], a[5], a[8]};
      } else {
        t[r] = {0.f, 0.f, 0.f, 0.f, 0.f, 0.f, 0.f, 0.f, 0.f};
      }
    }
    // row-0 transitions (begin and I_0), used by lane 0 of strip 0
    const float t0_mi = A.trans[1], t0_ii = A.trans[4];
    float M[kR], I[kR], D[kR];
#pragma unroll
    for (int r = 0; r < kR; ++r) M[r] = I[r] = D[r] = 0.f;
    int s = 0;                                  // my exponent (meaningful once `set`)
    bool set = false;                           // my values are all zero until the wavefront arrives
    float pM = 0.f, pI = 0.f, pD = 0.f;         // row above at my previous column (my scale)
    float m0 = 0.f, i0 = 0.f;                   // lane 0, strip 0: begin M_0 and I_0 (row 0) at the previous column
    int e0 = 0;                                 // their exponent
    const int steps = T + 1 + 31;
    const bool first_strip = st == 0;
    const bool last_strip_lane = lane == 31 && st + 1 < strips;
    const uint32_t em32 = (uint32_t)__cvta_generic_to_shared(em) + (uint32_t)((128 * st + lane) * 16);
    for (int k = 0; k < steps; ++k) {
      const int i = k - lane;
      const bool live = i >= 0 && i <= T;
      const int c = (i >= 1 && i <= T) ? (int)__ldg(x + i - 1) : K;  // x_i (1-based), dead outside
      // the row above at column i (lane l-1's values from its previous step) and its exponent
      float uM = __shfl_up_sync(0xffffffffu, M[kR - 1], 1);
      float uI = __shfl_up_sync(0xffffffffu, I[kR - 1], 1);
      float uD = __shfl_up_sync(0xffffffffu, D[kR - 1], 1);
      int us = __shfl_up_sync(0xffffffffu, s, 1);
      if (lane == 0) {
        if (first_strip) {
          // row 0 at column i: M_0(i) = [i == 0] (begin), I_0(i) = eI_0(x_i) (M_0(i-1) t0_MI + I_0(i-1) t0_II)
          const float ei0 = ei0t[c];
          const float ni0 = ei0 * fmaf(m0, t0_mi, i0 * t0_ii);
          const float nm0 = (i == 0) ? 1.0f : 0.f;   // e0 == 0 at i == 0
          m0 = nm0; i0 = ni0;
          // keep row 0 near 1 (it only decays)
          const float mx = fmaxf(m0, i0);
          if (mx > 0.f && mx < 1e-10f) {
            const int e = ilogbf(mx);
            m0 *= exp2i(-e); i0 *= exp2i(-e); e0 += e;
          }
          uM = m0; uI = i0; uD = 0.f; us = e0;
        } else {
          const float4 b = live ? bnd[i] : make_float4(0.f, 0.f, 0.f, 0.f);
          uM = b.x; uI = b.y; uD = b.z; us = live ? __float_as_int(b.w) : s;
        }
      }
      // scales: the first nonzero input fixes my exponent; a lane whose values are negligible next to
      // its input adopts the input's exponent (exact: a power-of-two rescale)
      if (!set && (uM != 0.f || uI != 0.f || uD != 0.f)) { s = us; set = true; }
      int d = us - s;
      if (d > 24) {
        const float f = exp2i(-d);
#pragma unroll
        for (int r = 0; r < kR; ++r) { M[r] *= f; I[r] *= f; D[r] *= f; }
        pM *= f; pI *= f; pD *= f;
        s = us;
        d = 0;
      }
      const float fin = exp2i(d);
      uM *= fin; uI *= fin; uD *= fin;
      // column i, rows j0 .. j0+7: the diagonal comes from (pM, pI, pD) then from my old row r-1
      float dM = pM, dI = pI, dD = pD;
      pM = uM; pI = uI; pD = uD;
      const uint32_t ea = em32 + (uint32_t)(c * S * 16);
#pragma unroll
      for (int r = 0; r < kR; r += 2) {
        float4 e;  // rows j0 + r, j0 + r + 1: chunk k = r / 2 at 32 k chunks
        asm("ld.shared.v4.f32 {%0, %1, %2, %3}, [%4];" : "=f"(e.x), "=f"(e.y), "=f"(e.z), "=f"(e.w) : "r"(ea + 256 * r));
#pragma unroll
        for (int h = 0; h < 2; ++h) {
          const int q = r + h;
          const float eM = h ? e.z : e.x, eI = h ? e.w : e.y;
          const float oM = M[q], oI = I[q], oD = D[q];
          const float nM = eM * fmaf(dM, t[q].mm, fmaf(dI, t[q].im, dD * t[q].dm));
          const float nI = eI * fmaf(oM, t[q].mi, fmaf(oI, t[q].ii, oD * t[q].di));
          const float nD = fmaf(uM, t[q].md, fmaf(uI, t[q].id, uD * t[q].dd));
          dM = oM; dI = oI; dD = oD;
          M[q] = nM; I[q] = nI; D[q] = nD;
          uM = nM; uI = nI; uD = nD;
        }
      }
      if (last_strip_lane && live) bnd[i] = make_float4(M[kR - 1], I[kR - 1], D[kR - 1], __int_as_float(s));
      // P(x) from the last row at column T
      if (i == T && st == strips - 1 && jL >= j0 && jL < j0 + kR) {
        const int q = jL - j0;
        float v = 0.f;
#pragma unroll
        for (int r = 0; r < kR; ++r)
          if (r == q) v = fmaf(M[r], A.trans[L * 9 + 0], fmaf(I[r], A.trans[L * 9 + 3], D[r] * A.trans[L * 9 + 6]));
        out_val = v; out_exp = s; have_out = true;
      }
      // renormalise to my maximum every 4 steps (exponents only move in whole powers of two)
      if ((k & 3) == 3 && set) {
        float mx = fmaxf(fmaxf(pM, pI), pD);
#pragma unroll
        for (int r = 0; r < kR; ++r) mx = fmaxf(mx, fmaxf(fmaxf(M[r], I[r]), D[r]));
        if (mx > 0.f && (mx < 0x1p-20f || mx > 0x1p20f)) {
          const int e = ilogbf(mx);
          const float f = exp2i(-e);
#pragma unroll
          for (int r = 0; r < kR; ++r) { M[r] *= f; I[r] *= f; D[r] *= f; }
          pM *= f; pI *= f; pD *= f;
          s += e;
        }
      }
    }
    __syncwarp();
  }
  if (have_out) A.ll_out[p] = out_val > 0.f ? logf(out_val) + (float)out_exp * 0.69314718055994531f : -INFINITY;
}

}  // namespace

// every lane's 8 rows of every strip are in the table (rows past L read zeros): 16-byte chunks
// per residue
int rows_tab_of(int L) { return ((L + kStripRows - 1) / kStripRows) * (kStripRows / 2); }

size_t phmm_smem_bytes(int L, int K, int64_t max_len) {
  const int strips = (L + kStripRows - 1) / kStripRows;
  size_t b = (size_t)(K + 1) * rows_tab_of(L) * sizeof(float4) + 128 * sizeof(float);
  if (strips > 1) b += (size_t)kPW * (size_t)(max_len + 1) * sizeof(float4);
  return b;
}

cudaError_t phmm_forward(const PhmmArgs& a, cudaStream_t s, int64_t* launches) {
  if (a.n == 0) return cudaSuccess;
  PhmmArgs A = a;
  A.rows_tab = rows_tab_of(A.L);
  const size_t smem = phmm_smem_bytes(A.L, A.K, A.max_len);
  cudaError_t e = cudaFuncSetAttribute(k_phmm_forward, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  ++*launches;
  k_phmm_forward<<<(unsigned)((A.n + kPW - 1) / kPW), kPW * 32, smem, s>>>(A);
  return cudaGetLastError();
}

}  // namespace dpk
