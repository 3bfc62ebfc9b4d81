// Affine-gap Smith–Waterman (Gotoh, DESIGN.md R-SW-AFFINE) packed:
// TWO problems per warp in the 16-bit halves of every register, like k_sw16 (sw16.cu) for the
// linear recursion. The schedule is the same (1,1) (the three tables' cross-cell offsets are the
// linear recursion's families); lane l owns rows [256 st + 8 l, +8) and works on column
// j = k - l + 1 at step k; H and F of the lane's last row move down the warp by __shfl_up_sync,
// E stays with its row.
//
// Cells are KEYS 4 v + code (s16x2), so the maxima the recurrence takes anyway also pick the
// traceback's tie-breaks (R-TB-SWA: in H diagonal > F > E; in E / F opening > extending):
//   E4 = (max(Ho(i,j-1), E4(i,j-1) - 4ge - 1) & ~3) | 1      (code 1 = open)
//   F4 = (max(Ho(i-1,j), F4(i-1,j) - 4ge - 2) & ~3) | 2
//   Hk = max(Ho(i-1,j-1) + s(a_i,b_j), F4, E4, 0)             (H code: 3 diag, 2 F, 1 E, 0 zero)
//   Ho = (Hk & ~3) + o,   o = -4(go+ge) + 1,   s = 4 sigma + 3 - o  (the profile holds s)
// E4 / F4 carry their H-source code in the low bits, and the extension constants take it off
// again; a cell is kept as Ho, the OPENING candidate of its right and lower neighbours, so one
// add serves both. Per packed cell: E 2 ops, F 2, the diagonal 1, H 3. The traceback retains 4 bits per cell and problem: the H code,
// F opened, E opened (one 32-bit word per lane, column and problem; one coalesced 64-bit store
// per step), walked by one thread per problem (k_affine16_tb) with the score tracked exactly.
// The end cell (first row-major maximum, R-TB-SW) comes from per-row running maxima and the
// column where each was first reached (a sign-select per row and step).
#include <algorithm>
#include <cstdint>
#include <type_traits>
#include <cuda_runtime.h>

#include "dp_internal.h"

namespace dpk {
namespace {

constexpr int kRows = 8;              // rows per lane
constexpr int kStrip = 32 * kRows;    // rows per strip
constexpr int kPad = 32;              // dead columns on each side of the column records
constexpr int kDead = -128;           // keyed profile value outside a problem (any negative value works)
constexpr uint32_t kClean = 0xfffcfffcu;

__device__ __forceinline__ uint32_t prmt(uint32_t a, uint32_t b, uint32_t sel) {
  uint32_t r;
  asm("prmt.b32 %0, %1, %2, %3;" : "=r"(r) : "r"(a), "r"(b), "r"(sel));
  return r;
}
template <int Q>
__device__ __forceinline__ uint32_t pack_sig(uint32_t wa, uint32_t wb) {  // {sext(a.byte Q), sext(b.byte Q)}
  constexpr uint32_t sel = (uint32_t)Q | ((8u | Q) << 4) | ((4u + Q) << 8) | ((8u | (4u + Q)) << 12);
  return prmt(wa, wb, sel);
}
template <uint32_t F>
__device__ __forceinline__ uint32_t lop3(uint32_t a, uint32_t b, uint32_t c) {
  uint32_t d;
  asm("lop3.b32 %0, %1, %2, %3, %4;" : "=r"(d) : "r"(a), "r"(b), "r"(c), "n"(F));
  return d;
}
// a * b + c on the FMA pipe (the ALU pipe is the bound here): ~x as x * -1 - 1 (the 32-bit identity
// holds for both halves at once), shifted merges of disjoint bit fields as multiply-adds
__device__ __forceinline__ uint32_t mad(uint32_t a, uint32_t b, uint32_t c) {
  uint32_t d;
  asm volatile("mad.lo.u32 %0, %1, %2, %3;" : "=r"(d) : "r"(a), "r"(b), "r"(c));
  return d;
}
__device__ __forceinline__ int lo16(uint32_t v) { return (int)(int16_t)(v & 0xffffu); }
__device__ __forceinline__ int hi16(uint32_t v) { return (int)(int16_t)(v >> 16); }
__device__ __forceinline__ uint32_t pk2(int v) { return (uint32_t)(uint16_t)(int16_t)v * 0x10001u; }
__device__ __forceinline__ uint32_t lds_u16(uint32_t a) {
  uint16_t v;
  asm("ld.shared.u16 %0, [%1];" : "=h"(v) : "r"(a));
  return v;
}
__device__ __forceinline__ uint2 lds_v2(uint32_t a) {
  uint2 v;
  asm("ld.shared.v2.u32 {%0, %1}, [%2];" : "=r"(v.x), "=r"(v.y) : "r"(a));
  return v;
}
__device__ __forceinline__ uint32_t lds_u32_v(uint32_t a) {
  uint32_t v;
  asm volatile("ld.shared.u32 %0, [%1];" : "=r"(v) : "r"(a) : "memory");
  return v;
}
__device__ __forceinline__ void sts_u32_v(uint32_t a, uint32_t v) {
  asm volatile("st.shared.u32 [%0], %1;" ::"r"(a), "r"(v) : "memory");
}

// nibble position of row r in a problem's code word (see the gather in aff_step)
__host__ __device__ __forceinline__ int nib_shift(int r) { return 8 * ((r & 1) + 2 * (r >> 2)) + 4 * ((r >> 1) & 1); }

template <bool MULTI>
__host__ __device__ constexpr int rec_bytes() { return MULTI ? 12 : 4; }  // u16 x 2 profile rows (+ H, F boundary)

struct AffState {
  uint32_t H[kRows];   // Ho = 4 H + o of my rows at my current column
  uint32_t E[kRows];   // E keys 4 E + 1
  uint32_t rb[kRows];  // TB: ~(per-row running maximum of Ho); score-only: rb[0] is the lane maximum of Ho
  uint32_t rc[kRows];  // TB: column where rb was first reached
  uint32_t prevH;      // H(row above my first row, j - 1)
  uint32_t F7;         // F key of my last row at my current column
};

struct AffK {          // packed constants
  uint32_t open, exte, extf, negf;  // o, -4ge - 1, -4ge - 2, F(0, j) = -inf
  uint32_t m1;                      // 0xffffffff through an opaque move
};

// One step of one lane. CHECK: ramp steps (j may lie outside 1..lbm; dead profile values make
// columns j <= 0 reproduce H = 0 and cells past the ends stay below the best live cell).
// Returns the two problems' code words (TB).
template <bool TB, bool CHECK, bool MULTI>
__device__ __forceinline__ uint2 aff_step(AffState& S, uint32_t rec, int j, uint32_t j2, int lbm, bool lane0,
                                          bool spill31, bool from_bnd, const AffK& C, uint32_t laneA,
                                          uint32_t laneB) {
  const bool live = !CHECK || (j >= 1 && j <= lbm);
  const uint32_t fH = __shfl_up_sync(0xffffffffu, S.H[kRows - 1], 1);
  const uint32_t fF = __shfl_up_sync(0xffffffffu, S.F7, 1);
  uint32_t Hup, Fup;
  if (MULTI) {  // only lane 0 reads the boundary words (lane 31 rewrites them a few steps later)
    uint32_t bh = C.open, bf = C.negf;
    if (lane0 && from_bnd && live) { bh = lds_u32_v(rec + 4); bf = lds_u32_v(rec + 8); }
    Hup = lane0 ? bh : fH;
    Fup = lane0 ? bf : fF;
  } else {
    Hup = lane0 ? C.open : fH;
    Fup = lane0 ? C.negf : fF;
  }
  const uint32_t Hd = S.prevH;
  S.prevH = Hup;
  const uint2 ca = lds_v2(laneA + lds_u16(rec));
  const uint2 cb = lds_v2(laneB + lds_u16(rec + 2));
  uint32_t sg[kRows];
  sg[0] = pack_sig<0>(ca.x, cb.x); sg[1] = pack_sig<1>(ca.x, cb.x);
  sg[2] = pack_sig<2>(ca.x, cb.x); sg[3] = pack_sig<3>(ca.x, cb.x);
  sg[4] = pack_sig<0>(ca.y, cb.y); sg[5] = pack_sig<1>(ca.y, cb.y);
  sg[6] = pack_sig<2>(ca.y, cb.y); sg[7] = pack_sig<3>(ca.y, cb.y);
  // off the column chain: E (left neighbour in the same row) and the diagonal term
  uint32_t Ek[kRows], E4[kRows], Xp[kRows];
#pragma unroll
  for (int r = 0; r < kRows; ++r) {
    Ek[r] = __viaddmax_s16x2(S.E[r], C.exte, S.H[r]);
    E4[r] = lop3<0xEA>(Ek[r], kClean, 0x00010001u);  // (Ek & ~3) | 1
    Xp[r] = __viaddmax_s16x2(r == 0 ? Hd : S.H[r - 1], sg[r], E4[r]);
  }
  // the column chain: F from the cell above, then H
  uint32_t hu = Hup, fu = Fup, nib[kRows / 2], Hk0 = 0, Fk0 = 0;
#pragma unroll
  for (int r = 0; r < kRows; ++r) {
    const uint32_t Fk = __viaddmax_s16x2(fu, C.extf, hu);
    const uint32_t F4 = lop3<0xEA>(Fk, kClean, 0x00020002u);  // (Fk & ~3) | 2
    const uint32_t Hk = __vimax3_s16x2(Xp[r], F4, 0u);
    const uint32_t Hc = __vadd2(Hk & kClean, C.open);         // Ho
    if (TB) {
      // codes: bytes {r-1 lo, r-1 hi, r lo, r hi} of the three keys, one nibble per byte
      if (r & 1) {
        const uint32_t wH = prmt(Hk0, Hk, 0x6420u), wF = prmt(Fk0, Fk, 0x6420u), wE = prmt(Ek[r - 1], Ek[r], 0x6420u);
        const uint32_t n = mad(wF & 0x01010101u, 4u, wH & 0x03030303u);
        nib[r >> 1] = mad(wE & 0x01010101u, 8u, n);
      }
      Hk0 = Hk; Fk0 = Fk;
      // first row-major maximum: the column where each row's maximum is first reached
      // rb holds ~max = -max - 1, so Hc + rb < 0 exactly when Hc <= max
      const uint32_t m = prmt(__vadd2(Hc, S.rb[r]), 0u, 0xbb99u);  // 0xffff where Hc <= max
      S.rc[r] = lop3<0xE2>(S.rc[r], m, j2);                        // (rc & m) | (j2 & ~m)
      S.rb[r] = __vmins2(S.rb[r], mad(Hc, C.m1, C.m1));  // ~Hc (C.m1 = -1, opaque: kept an IMAD)
    }
    S.H[r] = Hc;
    S.E[r] = E4[r];
    hu = Hc;
    fu = F4;
  }
  if (!TB) {
    S.rb[0] = __vimax3_s16x2(S.rb[0], S.H[0], S.H[1]);
    S.rb[0] = __vimax3_s16x2(S.rb[0], S.H[2], S.H[3]);
    S.rb[0] = __vimax3_s16x2(S.rb[0], S.H[4], S.H[5]);
    S.rb[0] = __vimax3_s16x2(S.rb[0], S.H[6], S.H[7]);
  }
  S.F7 = fu;
  if (MULTI && spill31 && live) { sts_u32_v(rec + 4, hu); sts_u32_v(rec + 8, fu); }
  if (!TB) return make_uint2(0, 0);
  // bytes [A0|A2<<4, B0|B2<<4, A1|A3<<4, B1|B3<<4] and the same for rows 4-7, then per problem
  const uint32_t x = mad(nib[1], 16u, nib[0]), y = mad(nib[3], 16u, nib[2]);
  return make_uint2(prmt(x, y, 0x6420u), prmt(x, y, 0x7531u));
}

template <bool TB, bool MULTI>
__global__ void __launch_bounds__(kWarps * 32, 2) k_affine16(AlignArgs A, int smem_per_warp) {
  extern __shared__ __align__(16) uint8_t smem[];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int asz = A.asz;
  const int goe = A.gap_open + A.gap_ext, ge = A.gap_ext;
  // keyed sigma transposed, sigT[c][a] = 4 sigma(a, c) + 3 - o (32 x 32 int8): kDead outside the
  // alphabet, so a = 31 is a dead residue and c = asz a dead column code
  int8_t* sigT = reinterpret_cast<int8_t*>(smem);
  constexpr int sig_bytes = 32 * 32;
  for (int q = threadIdx.x; q < 32 * 32; q += blockDim.x) {
    const int c = q >> 5, a = q & 31;
    sigT[q] = (c < asz && a < asz) ? (int8_t)(4 * A.sigma[a * asz + c] + 3 + 4 * goe - 1) : (int8_t)kDead;
  }
  __syncthreads();
  const int64_t grp = (int64_t)blockIdx.x * kWarps + warp;
  const int64_t pA = 2 * grp, pB = 2 * grp + 1;
  if (pA >= A.n) return;
  const bool hasB = pB < A.n;
  const int prof_bytes = (asz + 1) * kStrip;
  uint8_t* wbase = smem + sig_bytes + (size_t)warp * smem_per_warp;
  uint8_t* profA = wbase;
  uint8_t* profB = wbase + prof_bytes;
  constexpr int kRec = rec_bytes<MULTI>();
  const uint32_t sh_rec = (uint32_t)__cvta_generic_to_shared(wbase + 2 * prof_bytes);
  uint8_t* recg = wbase + 2 * prof_bytes;

  const uint8_t* aA = A.a_cat + A.a_off[pA];
  const uint8_t* bA = A.b_cat + A.b_off[pA];
  const int laA = (int)(A.a_off[pA + 1] - A.a_off[pA]);
  const int lbA = (int)(A.b_off[pA + 1] - A.b_off[pA]);
  const uint8_t* aB = hasB ? A.a_cat + A.a_off[pB] : aA;
  const uint8_t* bB = hasB ? A.b_cat + A.b_off[pB] : bA;
  const int laB = hasB ? (int)(A.a_off[pB + 1] - A.a_off[pB]) : 0;
  const int lbB = hasB ? (int)(A.b_off[pB + 1] - A.b_off[pB]) : 0;
  const int lbm = max(lbA, lbB), lam = max(laA, laB);
  if (lbm == 0 || lam == 0) {
    if (lane == 0) {
      A.scores[pA] = 0;
      if (hasB) A.scores[pB] = 0;
      if (TB) {
        A.ends[2 * pA] = A.ends[2 * pA + 1] = 0;
        if (hasB) A.ends[2 * pB] = A.ends[2 * pB + 1] = 0;
      }
    }
    return;
  }
  for (int q = lane; q < lbm + 2 * kPad; q += 32) {
    const int jj = q - kPad;  // 0-based column
    const int cA = (jj >= 0 && jj < lbA && laA > 0) ? bA[jj] : asz;
    const int cB = (jj >= 0 && jj < lbB && laB > 0) ? bB[jj] : asz;
    *reinterpret_cast<uint32_t*>(recg + q * kRec) = (uint32_t)(cA * kStrip) | ((uint32_t)(cB * kStrip) << 16);
  }
  AffK C;
  C.open = pk2(-4 * goe + 1);
  C.exte = pk2(-4 * ge - 1);
  C.extf = pk2(-4 * ge - 2);
  C.negf = pk2(-4 * (goe + 2) + 2);  // F(0, j) = -inf: below every opening (H = 0) after one extension
  asm volatile("mov.b32 %0, %1;" : "=r"(C.m1) : "r"(0xffffffffu));
  const uint32_t nege = pk2(-4 * (goe + 2) + 1);  // E(i, 0) = -inf
  const int strips = (lam + kStrip - 1) / kStrip;
  const uint32_t laneA = (uint32_t)__cvta_generic_to_shared(profA) + lane * kRows;
  const uint32_t laneB = (uint32_t)__cvta_generic_to_shared(profB) + lane * kRows;
  const bool lane0 = lane == 0;
  // per half: best, its row and column (first row-major maximum)
  int bestv[2] = {0, 0}, besti[2] = {0, 0}, bestj[2] = {0, 0};
  uint32_t lanemax = C.open;
  AffState S;

  for (int st = 0; st < strips; ++st) {
    const int i0 = st * kStrip + lane * kRows;  // 0-based index of my first row
    // profiles for my 8 rows (as k_sw16): each 4-row word gathered from column c of sigT by byte
    // permutes, residue a selecting byte a & 7 of window a >> 3
    uint32_t sel[4], msk[4][4];
#pragma unroll
    for (int g4 = 0; g4 < 4; ++g4) {
      const uint8_t* src = g4 < 2 ? aA : aB;
      const int la = g4 < 2 ? laA : laB;
      uint32_t sl = 0, m[4] = {0, 0, 0, 0};
#pragma unroll
      for (int k = 0; k < 4; ++k) {
        const int i = i0 + 4 * (g4 & 1) + k;
        const int a = i < la ? src[i] : 31;  // dead rows read kDead
        sl |= (uint32_t)(a & 7) << (4 * k);
        m[a >> 3] |= 0xffu << (8 * k);
      }
      sel[g4] = sl;
#pragma unroll
      for (int w = 0; w < 4; ++w) msk[g4][w] = m[w];
    }
    for (int c = 0; c <= asz; ++c) {
      uint32_t col[8];
      const uint4 c0 = *reinterpret_cast<const uint4*>(sigT + 32 * c);
      const uint4 c1 = *reinterpret_cast<const uint4*>(sigT + 32 * c + 16);
      col[0] = c0.x; col[1] = c0.y; col[2] = c0.z; col[3] = c0.w;
      col[4] = c1.x; col[5] = c1.y; col[6] = c1.z; col[7] = c1.w;
      uint32_t w[4];
#pragma unroll
      for (int g4 = 0; g4 < 4; ++g4) {
        uint32_t v = prmt(col[0], col[1], sel[g4]) & msk[g4][0];
#pragma unroll
        for (int win = 1; win < 4; ++win) v |= prmt(col[2 * win], col[2 * win + 1], sel[g4]) & msk[g4][win];
        w[g4] = v;
      }
      *reinterpret_cast<uint2*>(profA + c * kStrip + lane * kRows) = make_uint2(w[0], w[1]);
      *reinterpret_cast<uint2*>(profB + c * kStrip + lane * kRows) = make_uint2(w[2], w[3]);
    }
    __syncwarp();
#pragma unroll
    for (int r = 0; r < kRows; ++r) { S.H[r] = C.open; S.E[r] = nege; S.rb[r] = TB ? ~C.open : C.open; S.rc[r] = 0; }
    S.prevH = C.open; S.F7 = C.negf;
    const bool from_bnd = st > 0;
    const bool spill31 = (st + 1 < strips) && lane == 31;
    uint2* cds = TB ? reinterpret_cast<uint2*>(A.dirs + grp * A.dir_stride) + (int64_t)st * A.max_lb * 32 + lane - 32
                    : nullptr;  // word pair of column j at cds + 32 j
    const uint32_t rec0 = sh_rec + kRec * (kPad - lane);
    const int K = lbm + 31;
    // steady range: lane 31 at j >= 1 and lane 0 at j <= lbm - 1
    const int s0 = min(31, K), s1 = max(s0, lbm - 1);
    constexpr int U = 8;
    int k = 0;
    auto one = [&](auto chk, int kk) {
      constexpr bool CH = decltype(chk)::value;
      const int j = kk - lane + 1;
      const uint2 cw = aff_step<TB, CH, MULTI>(S, rec0 + kRec * kk, j, (uint32_t)(uint16_t)j * 0x10001u, lbm, lane0,
                                               spill31, from_bnd, C, laneA, laneB);
      if (TB && (!CH || (j >= 1 && j <= lbm))) cds[32 * j] = cw;
    };
    for (; k < s0; ++k) {
      one(std::true_type(), k);
      // lane 0 reads column j's boundary words at step j - 1, lane 31 rewrites them at step j + 30
      if (MULTI) __syncwarp();
    }
    for (; k + U <= s1; k += U) {
#pragma unroll
      for (int u = 0; u < U; ++u) one(std::false_type(), k + u);
      if (MULTI) __syncwarp();
    }
    for (; k < s1; ++k) {
      one(std::false_type(), k);
      if (MULTI) __syncwarp();
    }
    for (; k < K; ++k) {
      one(std::true_type(), k);
      if (MULTI) __syncwarp();
    }
    if (TB) {
#pragma unroll
      for (int r = 0; r < kRows; ++r) {
#pragma unroll
        for (int h = 0; h < 2; ++h) {
          const uint32_t mx = ~S.rb[r];
          const int v = ((h ? hi16(mx) : lo16(mx)) + 4 * goe - 1) >> 2;
          if (v > bestv[h]) { bestv[h] = v; besti[h] = i0 + r + 1; bestj[h] = h ? hi16(S.rc[r]) : lo16(S.rc[r]); }
        }
      }
    } else {
      lanemax = __vmaxs2(lanemax, S.rb[0]);
    }
    __syncwarp();
  }
  if (TB) {
#pragma unroll
    for (int h = 0; h < 2; ++h) {
      int b = bestv[h], bi = besti[h], bj = bestj[h];
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) {  // max value, then smallest i, then smallest j
        const int ob = __shfl_xor_sync(0xffffffffu, b, o);
        const int oi = __shfl_xor_sync(0xffffffffu, bi, o);
        const int oj = __shfl_xor_sync(0xffffffffu, bj, o);
        if (ob > b || (ob == b && (oi < bi || (oi == bi && oj < bj)))) { b = ob; bi = oi; bj = oj; }
      }
      const int64_t p = h ? pB : pA;
      if (lane == 0 && (h == 0 || hasB)) {
        A.scores[p] = b;
        A.ends[2 * p] = b > 0 ? bi : 0;
        A.ends[2 * p + 1] = b > 0 ? bj : 0;
      }
    }
  } else {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) lanemax = __vmaxs2(lanemax, __shfl_xor_sync(0xffffffffu, lanemax, o));
    if (lane == 0) {
      A.scores[pA] = (lo16(lanemax) + 4 * goe - 1) >> 2;
      if (hasB) A.scores[pB] = (hi16(lanemax) + 4 * goe - 1) >> 2;
    }
  }
}

// One thread per problem walks the three-state machine back from the end cell (R-TB-SWA), the
// value in the current state tracked exactly; the H code is the key code (3 diag, 2 F, 1 E).
__global__ void __launch_bounds__(128) k_affine16_tb(AlignArgs A, int64_t first, int64_t count, uint8_t* out,
                                                     int64_t stride, int32_t* out_len, int32_t* coords) {
  const int64_t q = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (q >= count) return;
  const int64_t p = first + q;
  const uint8_t* a = A.a_cat + A.a_off[p];
  const uint8_t* b = A.b_cat + A.b_off[p];
  const uint32_t* dirp = A.dirs + (p >> 1) * A.dir_stride + (p & 1);
  const int ei = A.ends[2 * p], ej = A.ends[2 * p + 1];
  const int ge = A.gap_ext, goe = A.gap_open + A.gap_ext;
  auto code_at = [&](int i, int j) -> uint32_t {
    const int row = i - 1, st = row / kStrip, lane = (row % kStrip) / kRows, r = row % kRows;
    const uint32_t w = __ldg(dirp + (((int64_t)st * A.max_lb + (j - 1)) * 32 + lane) * 2);
    return (w >> nib_shift(r)) & 15u;
  };
  int i = ei, j = ej, v = A.scores[p], state = 0;  // v = H (state 0), F (1) or E (2) at (i, j)
  uint8_t* o = out + q * stride;
  int64_t nops = 0;
  bool overflow = false;
  while (!(state == 0 && v <= 0)) {
    const uint32_t c = code_at(i, j);
    uint8_t op;
    if (state == 0) {
      const uint32_t src = c & 3u;
      if (src == 3u) {
        op = (a[i - 1] == b[j - 1]) ? 'M' : 'X';
        v -= A.sigma[a[i - 1] * A.asz + b[j - 1]];
        --i; --j;
      } else {
        state = src == 2u ? 1 : 2;  // H(i,j) == F(i,j) or E(i,j): same value, no move
        continue;
      }
    } else if (state == 1) {
      op = 'D';
      if (c & 4u) { state = 0; v += goe; } else { v += ge; }
      --i;
    } else {
      op = 'I';
      if (c & 8u) { state = 0; v += goe; } else { v += ge; }
      --j;
    }
    if (nops < stride) o[nops] = op; else overflow = true;
    ++nops;
  }
  if (!overflow)
    for (int64_t u = 0, w = nops - 1; u < w; ++u, --w) { const uint8_t t = o[u]; o[u] = o[w]; o[w] = t; }
  out_len[q] = overflow ? -1 : (int32_t)nops;
  if (coords) {
    coords[4 * q] = i; coords[4 * q + 1] = j; coords[4 * q + 2] = ei; coords[4 * q + 3] = ej;
  }
}

int affine16_per_warp(int asz, int64_t max_la, int64_t max_lb) {
  const int rec = max_la > kStrip ? rec_bytes<true>() : rec_bytes<false>();
  return (int)((2 * (asz + 1) * kStrip + (max_lb + 2 * kPad) * rec + 15) & ~int64_t(15));
}

template <bool TB, bool MULTI>
cudaError_t launch16(const AlignArgs& A, cudaStream_t s) {
  const int per_warp = affine16_per_warp(A.asz, A.max_la, A.max_lb);
  const size_t smem = 32 * 32 + (size_t)kWarps * per_warp;
  auto kern = k_affine16<TB, MULTI>;
  cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  e = cudaFuncSetAttribute(kern, cudaFuncAttributePreferredSharedMemoryCarveout, 100);
  if (e != cudaSuccess) return e;
  const int64_t groups = (A.n + 1) / 2;
  kern<<<(unsigned)((groups + kWarps - 1) / kWarps), kWarps * 32, smem, s>>>(A, per_warp);
  return cudaGetLastError();
}

}  // namespace

bool affine16_eligible(int64_t max_la, int64_t max_lb, const int8_t* sigma_host, int asz, int go, int ge) {
  int smax = 0, smin = 0;
  for (int q = 0; q < asz * asz; ++q) { smax = std::max(smax, (int)sigma_host[q]); smin = std::min(smin, (int)sigma_host[q]); }
  const int64_t bound = (int64_t)smax * std::min(max_la, max_lb);  // H <= bound
  // keys 4 v + 3 in int16: 4 bound; E, F >= -(go + ge) after one opening; the -inf keys
  // -4 (go + ge + 2) minus one extension
  // profile 4 sigma + 3 - o = 4 sigma + 4 (go + ge) + 2 in int8
  return asz < 32 && 4 * smax + 4 * (go + ge) + 2 <= 127 && 4 * smin + 4 * (go + ge) + 2 >= -127 &&
         4 * bound + 3 <= 32000 && go >= 0 && ge >= 1 && 4 * (go + 2 * ge + 3) <= 32000 && max_lb <= 32000;
}

size_t affine16_smem_bytes(int asz, int64_t max_la, int64_t max_lb) {
  return 32 * 32 + (size_t)kWarps * (size_t)affine16_per_warp(asz, max_la, max_lb);
}

int64_t affine16_dir_words(int64_t max_la, int64_t max_lb) {  // per GROUP of two problems
  return ((max_la + kStrip - 1) / kStrip) * max_lb * 64;
}

cudaError_t affine16_solve(const AlignArgs& A, cudaStream_t s, int64_t* launches) {
  if (A.n == 0) return cudaSuccess;
  ++*launches;
  const bool tb = A.dirs != nullptr, multi = A.max_la > kStrip;
  return tb ? (multi ? launch16<true, true>(A, s) : launch16<true, false>(A, s))
            : (multi ? launch16<false, true>(A, s) : launch16<false, false>(A, s));
}

cudaError_t affine16_traceback(const AlignArgs& A, int64_t first, int64_t count, uint8_t* out, int64_t stride,
                               int32_t* out_len, int32_t* coords, cudaStream_t s, int64_t* launches) {
  if (count == 0) return cudaSuccess;
  ++*launches;
  k_affine16_tb<<<(unsigned)((count + 127) / 128), 128, 0, s>>>(A, first, count, out, stride, out_len, coords);
  return cudaGetLastError();
}

}  // namespace dpk
