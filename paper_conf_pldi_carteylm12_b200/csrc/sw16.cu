// Smith–Waterman (§6.1, linear gap) on the anti-diagonal schedule
// (1,1), packed: TWO problems per warp in the two 16-bit halves of every
// register (VIADDMNMX.S16x2 / VIMNMX3.S16x2), legal because scores stay below
// 2^15 (max sigma x min length; checked by the plan).
//
// Layout of the sweep (as in align.cu): lane l owns rows [256 st + 8l, +8),
// step k works on column j = k - l + 1 (tiles of 8 rows x 1 column under the
// schedule (1,1)); the boundary row moves down the warp by __shfl_up_sync.
// Cells are kept in "gap-shifted" form G = H - g, so that
//     G(i,j) = max(G(i-1,j) - g, X),  X = max(G(i-1,j-1) + sigma(a_i,b_j), G(i,j-1) - g, -g)
// (three VIADDMNMX.S16x2 per packed cell, only ONE of them on the dependence
// chain down the column), with the per-problem profile P[c][i] = sigma(a_i, c)
// (int8, shared memory) merged into s16x2 by one PRMT (sign-replicating selector).
// Steps run in blocks of 32; inside a block the steady steps (every lane inside
// the table) carry no bounds checks, the ramp steps compute dead cells instead
// of branching.
//
// Traceback retention without per-cell direction codes: the forward pass
// stores checkpoints of G — the bottom row of every 16-row band (odd lanes,
// every column) and, after every block of 32 steps, every lane's 8 rows at the
// column it is on (a staircase, column 32 s - lane: warp-uniform, coalesced,
// no per-step branch), the G above it there and its best G over the block
// (0.25 B/cell). k_sw16_tb2 recomputes only the 32x32 (sheared) blocks the
// canonical traceback needs and walks them with the oracle's tie-break
// (diag > up > left, stop at H = 0; end cell = first maximum in row-major order).
#include <cstdint>
#include <cstdlib>
#include <cuda_runtime.h>

#include "dp_internal.h"

namespace dpk {
namespace {

constexpr int kRows = 8;              // rows per lane
constexpr int kStrip = 32 * kRows;    // rows per strip
constexpr int kBand = 16;             // checkpoint band height (two lanes)
constexpr int kLanesPerBand = kBand / kRows;
constexpr int kBandsPerStrip = kStrip / kBand;
constexpr int kBlk = 32;              // traceback recompute block height (two independent bands)
constexpr int kSlab = 32;             // checkpoint column spacing
constexpr int kDead = -100;           // profile value for rows/columns outside a problem
constexpr int kPad = 32;              // dead columns on each side of the residue array

__device__ __forceinline__ uint32_t prmt(uint32_t a, uint32_t b, uint32_t sel) {
  uint32_t r;
  asm("prmt.b32 %0, %1, %2, %3;" : "=r"(r) : "r"(a), "r"(b), "r"(sel));
  return r;
}
// s16x2 {sext(a.byte q), sext(b.byte q)}
template <int Q>
__device__ __forceinline__ uint32_t pack_sig(uint32_t wa, uint32_t wb) {
  constexpr uint32_t sel = (uint32_t)Q | ((8u | Q) << 4) | ((4u + Q) << 8) | ((8u | (4u + Q)) << 12);
  return prmt(wa, wb, sel);
}
__device__ __forceinline__ int lo16(uint32_t v) { return (int)(int16_t)(v & 0xffffu); }
__device__ __forceinline__ int hi16(uint32_t v) { return (int)(int16_t)(v >> 16); }
__device__ __forceinline__ int half16(uint32_t v, int h) { return h ? hi16(v) : lo16(v); }

struct FwdState {
  uint32_t G[kRows];
  uint32_t prev, bbest, best2;
};

// shared-space accessors (32-bit shared addresses; the read-only profile and
// column records are plain asm so the scheduler may move them, the boundary
// word handed from lane 31 to lane 0 is volatile)
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

// Per-column record in shared memory (column q = j + kPad - 1):
//   u16 byte offset of problem A's profile row for b_A[j] (dead code outside A),
//   u16 the same for problem B, and (multi-strip sweeps only) the u32 boundary
//   word G(256 st, j) handed from lane 31 of strip st-1 to lane 0 of strip st.
template <bool MULTI>
__host__ __device__ constexpr int rec_bytes() { return MULTI ? 8 : 4; }

// Checkpoint pointers of one lane (TB only).
// One step of the sweep for one lane. `rec` = record address of this lane's
// column j. CHECK: ramp steps, where j may lie outside 1..lbm (computed with dead
// profile values: columns j <= 0 reproduce the boundary G = -g exactly, cells
// past the end stay strictly below the best live cell; stores suppressed).
template <bool TB, bool CHECK, bool MULTI>
__device__ __forceinline__ void sw_step(FwdState& S, uint32_t rec, int j, int lbm, bool lane0, bool odd, bool spill31,
                                        bool from_bnd, uint32_t NEG_G2, uint32_t laneA, uint32_t laneB,
                                        uint32_t* rk) {
  const bool live = !CHECK || (j >= 1 && j <= lbm);
  const uint32_t fa = __shfl_up_sync(0xffffffffu, S.G[kRows - 1], 1);
  uint32_t Gu;
  if (MULTI) {
    const uint32_t bw = lds_u32_v(rec + 4);
    Gu = lane0 ? ((from_bnd && live) ? bw : NEG_G2) : fa;
  } else {
    Gu = lane0 ? NEG_G2 : fa;
  }
  const uint32_t Gd = S.prev;
  S.prev = Gu;
  const uint2 ca = lds_v2(laneA + lds_u16(rec));
  const uint2 cb = lds_v2(laneB + lds_u16(rec + 2));
  uint32_t sg[kRows];
  sg[0] = pack_sig<0>(ca.x, cb.x); sg[1] = pack_sig<1>(ca.x, cb.x);
  sg[2] = pack_sig<2>(ca.x, cb.x); sg[3] = pack_sig<3>(ca.x, cb.x);
  sg[4] = pack_sig<0>(ca.y, cb.y); sg[5] = pack_sig<1>(ca.y, cb.y);
  sg[6] = pack_sig<2>(ca.y, cb.y); sg[7] = pack_sig<3>(ca.y, cb.y);
  // off the critical path: X_r = max(G(i-1,j-1) + sigma, G(i,j-1) - g, -g)
  uint32_t X[kRows];
  X[0] = __viaddmax_s16x2(Gd, sg[0], __viaddmax_s16x2(S.G[0], NEG_G2, NEG_G2));
#pragma unroll
  for (int r = 1; r < kRows; ++r) X[r] = __viaddmax_s16x2(S.G[r - 1], sg[r], __viaddmax_s16x2(S.G[r], NEG_G2, NEG_G2));
  // the only dependence down the column: G(i,j) = max(G(i-1,j) - g, X)
  uint32_t g = Gu;
#pragma unroll
  for (int r = 0; r < kRows; ++r) {
    g = __viaddmax_s16x2(g, NEG_G2, X[r]);
    S.G[r] = g;
  }
  S.bbest = __vimax3_s16x2(S.bbest, S.G[0], S.G[1]);
  S.bbest = __vimax3_s16x2(S.bbest, S.G[2], S.G[3]);
  S.bbest = __vimax3_s16x2(S.bbest, S.G[4], S.G[5]);
  S.bbest = __vimax3_s16x2(S.bbest, S.G[6], S.G[7]);
  if (MULTI && spill31 && live) sts_u32_v(rec + 4, g);
  if (TB && odd && live) *rk = g;  // bottom row of a 16-row band, column j
}

template <bool TB, bool MULTI>
__global__ void __launch_bounds__(kWarps * 32, 2) k_sw16(Sw16Args A) {
  extern __shared__ __align__(16) uint8_t smem[];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int asz = A.asz, gap = A.gap;
  int8_t* sig_s = reinterpret_cast<int8_t*>(smem);
  const int sig_bytes = (asz * asz + 15) & ~15;
  for (int q = threadIdx.x; q < asz * asz; q += blockDim.x) sig_s[q] = A.sigma[q];
  __syncthreads();
  const int64_t grp = (int64_t)blockIdx.x * kWarps + warp;
  const int64_t pA = 2 * grp, pB = 2 * grp + 1;
  if (pA >= A.n) return;
  const bool hasB = pB < A.n;
  const int prof_bytes = (asz + 1) * kStrip;
  uint8_t* wbase = smem + sig_bytes + (size_t)warp * A.smem_per_warp;
  uint8_t* profA = wbase;
  uint8_t* profB = wbase + prof_bytes;
  // column records: 256-byte aligned in the shared window
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
    if (lane == 0) { A.scores[pA] = 0; if (hasB) A.scores[pB] = 0; }
    return;
  }
  // profile row offsets of each column; dead code `asz` outside each problem
  // and in the kPad columns on either side
  for (int q = lane; q < lbm + 2 * kPad; q += 32) {
    const int jj = q - kPad;  // 0-based column
    const int cA = (jj >= 0 && jj < lbA && laA > 0) ? bA[jj] : asz;
    const int cB = (jj >= 0 && jj < lbB && laB > 0) ? bB[jj] : asz;
    *reinterpret_cast<uint32_t*>(recg + q * kRec) = (uint32_t)(cA * kStrip) | ((uint32_t)(cB * kStrip) << 16);
  }
  const uint32_t NEG_G2 = (uint32_t)(uint16_t)(-gap) * 0x10001u;
  const int strips = (lam + kStrip - 1) / kStrip;
  const uint32_t laneA = (uint32_t)__cvta_generic_to_shared(profA) + lane * kRows;
  const uint32_t laneB = (uint32_t)__cvta_generic_to_shared(profB) + lane * kRows;
  const bool lane0 = lane == 0, odd = (lane & 1) != 0;
  FwdState S;
  S.best2 = NEG_G2;  // max G = max h - g

  for (int st = 0; st < strips; ++st) {
    const int i0 = st * kStrip + lane * kRows;  // 0-based index of my first row
    // profiles for my 8 rows: P[c][row] int8, one 8-byte word per lane per residue
    int ra[kRows], rb[kRows];
#pragma unroll
    for (int r = 0; r < kRows; ++r) {
      ra[r] = (i0 + r < laA) ? aA[i0 + r] : -1;
      rb[r] = (i0 + r < laB) ? aB[i0 + r] : -1;
    }
    for (int c = 0; c <= asz; ++c) {
      uint32_t w[4] = {0, 0, 0, 0};
#pragma unroll
      for (int r = 0; r < kRows; ++r) {
        const int va = (ra[r] >= 0 && c < asz) ? sig_s[ra[r] * asz + c] : kDead;
        const int vb = (rb[r] >= 0 && c < asz) ? sig_s[rb[r] * asz + c] : kDead;
        w[r / 4] |= (uint32_t)(uint8_t)(int8_t)va << (8 * (r % 4));
        w[2 + r / 4] |= (uint32_t)(uint8_t)(int8_t)vb << (8 * (r % 4));
      }
      *reinterpret_cast<uint2*>(profA + c * kStrip + lane * kRows) = make_uint2(w[0], w[1]);
      *reinterpret_cast<uint2*>(profB + c * kStrip + lane * kRows) = make_uint2(w[2], w[3]);
    }
    __syncwarp();
#pragma unroll
    for (int r = 0; r < kRows; ++r) S.G[r] = NEG_G2;  // column 0: H = 0
    S.prev = NEG_G2; S.bbest = NEG_G2;
    const bool from_bnd = st > 0;
    const bool spill31 = (st + 1 < strips) && lane == 31;
    uint32_t *rowck = nullptr, *colck = nullptr, *slab = nullptr, *corner = nullptr;
    if (TB) {
      rowck = A.rowck + ((grp * A.strips_max + st) * kBandsPerStrip + lane / kLanesPerBand) * A.max_lb;
      colck = A.colck + ((grp * A.strips_max + st) * A.nslab_max) * kStrip + lane * kRows;
      const int64_t sb = ((grp * A.strips_max + st) * A.nslab_max) * 32 + lane;
      slab = A.slabbest + sb;
      corner = A.corner + sb;
    }
    // step k works on column j = k - lane + 1, record address sh_rec + kRec (k - lane + kPad).
    // Steps come in blocks of 32 (one slab); after block s every lane checkpoints
    // at once (warp-uniform, coalesced): its 8 G values at column 32(s+1) - lane,
    // the G above it there (corner), and its best G over the block.
    const uint32_t rec0 = sh_rec + kRec * (kPad - lane);
    const int K = lbm + 31;
    constexpr int U = 4;
    for (int kb = 0, sl = 0; kb < K; kb += kSlab, ++sl) {
      const int ke = min(kb + kSlab, K);
      // steady range: lane 31 at j >= 1 and lane 0 at j <= lbm - 1
      const int s0 = min(max(kb, 31), ke), s1 = max(s0, min(ke, lbm - 1));
      int k = kb;
      for (; k < s0; ++k)
        sw_step<TB, true, MULTI>(S, rec0 + kRec * k, k - lane + 1, lbm, lane0, odd, spill31, from_bnd, NEG_G2,
                                 laneA, laneB, rowck + (k - lane));
      for (; k + U <= s1; k += U) {
        const uint32_t rec = rec0 + kRec * k;
        uint32_t* rk = rowck + (k - lane);
#pragma unroll
        for (int u = 0; u < U; ++u)
          sw_step<TB, false, MULTI>(S, rec + kRec * u, k + u - lane + 1, lbm, lane0, odd, spill31, from_bnd, NEG_G2,
                                    laneA, laneB, rk + u);
        if (MULTI) __syncwarp();
      }
      for (; k < s1; ++k)
        sw_step<TB, false, MULTI>(S, rec0 + kRec * k, k - lane + 1, lbm, lane0, odd, spill31, from_bnd, NEG_G2,
                                  laneA, laneB, rowck + (k - lane));
      for (; k < ke; ++k) {
        sw_step<TB, true, MULTI>(S, rec0 + kRec * k, k - lane + 1, lbm, lane0, odd, spill31, from_bnd, NEG_G2,
                                 laneA, laneB, rowck + (k - lane));
        if (MULTI) __syncwarp();
      }
      if (TB) {
        uint4* col = reinterpret_cast<uint4*>(colck + (int64_t)sl * kStrip);
        col[0] = make_uint4(S.G[0], S.G[1], S.G[2], S.G[3]);
        col[1] = make_uint4(S.G[4], S.G[5], S.G[6], S.G[7]);
        slab[sl * 32] = S.bbest;
        corner[sl * 32] = S.prev;
        S.best2 = __vmaxs2(S.best2, S.bbest);
        S.bbest = NEG_G2;
      }
    }
    S.best2 = __vmaxs2(S.best2, S.bbest);
    __syncwarp();
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) S.best2 = __vmaxs2(S.best2, __shfl_xor_sync(0xffffffffu, S.best2, o));
  if (lane == 0) {
    A.scores[pA] = lo16(S.best2) + gap;
    if (hasB) A.scores[pB] = hi16(S.best2) + gap;
  }
}

// ---------------------------------------------------------------- traceback
// Two problems per warp (the pair group of the forward pass): lanes 0-15 serve
// problem 2g, lanes 16-31 problem 2g+1. A 32-row block is recomputed by 16 lanes,
// lane hl holding block rows hl+1 (low half) and hl+17 (high half) in one s16x2
// register: the two halves are independent given the checkpoint row between them.
//
// The checkpoints are staircases: forward lane l (rows 8l+1..8l+8 of its strip)
// stored its column at 32 s - l. Block (blk, slab) therefore covers, for the
// rows of forward lane l = L0 + m (L0 = 4 (blk mod 8), m = 0..3), the columns
// j = D + c - m, c = 1..32, D = 32 slab - L0: a 32 x 32 square in the sheared
// column c. Inside one forward lane the recurrence keeps its shape; at the first
// row of lanes L0+1 and L0+3 (block rows 9 and 25: lane hl = 8 of each half) the
// row above sits one sheared column to the left, so "up" arrives one wavefront
// step later and the diagonal of the first column is the corner word the
// forward lane stored next to its checkpoint.
// Hp[t][c+1] packs (H of block row t, H of block row 16+t), c = -1..32. Row 0
// holds the checkpoint rows aligned with rows 1 and 17 (shear 0 and 2), column
// c = 0 the checkpoint columns, column c = -1 of row 8 the corners.
constexpr int kPS = kSlab + 2;        // packed row stride (words)
constexpr int kPW = 17 * kPS + 14;    // words per packed block (592 = 16 mod 32: the halves hit disjoint banks)

struct PackedView {
  const Sw16Args* A;
  int64_t grp;
  int half, la, lb;
  __device__ __forceinline__ int top_h(int band, int j) const {  // H at row 16*band, column j (0 off the table)
    if (band == 0 || j <= 0 || j > lb) return 0;
    const int b = band - 1;
    const int st = b / kBandsPerStrip, bi = b % kBandsPerStrip;
    const uint32_t v = A->rowck[((grp * A->strips_max + st) * kBandsPerStrip + bi) * A->max_lb + (j - 1)];
    return half16(v, half) + A->gap;
  }
  // H at row i, at its forward lane's checkpoint slab-1 (column 32 slab - lane)
  __device__ __forceinline__ int left_h(int i, int slab) const {
    if (slab == 0) return 0;
    const int st = (i - 1) / kStrip, ri = (i - 1) % kStrip;
    const uint32_t v = A->colck[((grp * A->strips_max + st) * A->nslab_max + (slab - 1)) * kStrip + ri];
    return half16(v, half) + A->gap;
  }
  // H of the row above forward lane `ln` (strip st) at its checkpoint slab-1
  __device__ __forceinline__ int corner_h(int st, int ln, int slab) const {
    if (slab == 0) return 0;
    const uint32_t v = A->corner[((grp * A->strips_max + st) * A->nslab_max + (slab - 1)) * 32 + ln];
    return half16(v, half) + A->gap;
  }
};

__device__ __forceinline__ uint32_t pk(int lo, int hi) { return (uint32_t)(uint16_t)lo | ((uint32_t)(uint16_t)hi << 16); }
// H of packed row t (0..16) of half hf at sheared column c (-1..32)
__device__ __forceinline__ int hp_at(const uint32_t* Hp, int hf, int t, int c) {
  const uint32_t v = Hp[t * kPS + c + 1];
  return hf ? hi16(v) : lo16(v);
}
// shear of packed row t of half hf (row 0 is aligned with row 1)
__device__ __forceinline__ int shear_of(int hf, int t) { return 2 * hf + (t >= 1 ? (t - 1) >> 3 : 0); }

constexpr int kDeadCode = 31;   // residue code whose sigma row/column is kDead (alphabets < 32)
constexpr int kBPadLo = 64, kBPadHi = 96;  // dead residues staged around b (the sheared sweep reads past both ends)

__device__ __forceinline__ int lds_s8(uint32_t a) {
  int v;
  asm("ld.shared.s8 %0, [%1];" : "=r"(v) : "r"(a));
  return v;
}
__device__ __forceinline__ uint32_t lds_u8(uint32_t a) {
  uint32_t v;
  asm("ld.shared.u8 %0, [%1];" : "=r"(v) : "r"(a));
  return v;
}

// Recompute this problem's block (blk, slab) into Hp; `on` = this half-warp has a
// block to do. sig32 = shared sigma with row stride 32 (kDead outside the
// alphabet); b is staged with kDeadCode padding, so columns j <= 0 evaluate to
// exactly H = 0 (the table border) without masks, and columns past lb (never
// read by the walk or the end-cell search) need none either.
__device__ void packed_block(const PackedView& V, const uint8_t* a, const uint8_t* b, int blk, int slab, bool on,
                             uint32_t* Hp, uint32_t sig32, int g, int hl) {
  const int R0 = blk * kBlk, st = R0 / kStrip, L0 = (R0 % kStrip) / kRows;
  const int D = slab * kSlab - L0;
  const int band0 = R0 / kBand;
  if (on) {
    for (int c = hl; c <= kSlab; c += 16)
      Hp[c + 1] = pk(V.top_h(band0, D + c), V.top_h(band0 + 1, D + c - 2));
  }
  const int mL = hl >> 3, mH = 2 + (hl >> 3);
  const int iL = R0 + hl + 1, iH = R0 + hl + 17;
  const bool okL = on && iL <= V.la, okH = on && iH <= V.la;
  uint32_t left = pk(okL ? V.left_h(iL, slab) : 0, okH ? V.left_h(iH, slab) : 0);
  if (on) Hp[(hl + 1) * kPS + 1] = left;
  const bool shear = hl == 8;
  uint32_t corner = 0;
  if (shear && on) {
    corner = pk(V.corner_h(st, L0 + 1, slab), V.corner_h(st, L0 + 3, slab));
    Hp[8 * kPS] = corner;
  }
  __syncwarp();
  const uint32_t sLa = sig32 + 32 * (okL ? a[iL - 1] : kDeadCode);
  const uint32_t sHa = sig32 + 32 * (okH ? a[iH - 1] : kDeadCode);
  const uint32_t bsh = (uint32_t)__cvta_generic_to_shared(b);
  const uint32_t bL = bsh + (D - mL - 1), bH = bsh + (D - mH - 1);  // residue of sheared column c at +c
  const uint32_t NEG_G2 = (uint32_t)(uint16_t)(-g) * 0x10001u;
  uint32_t* hrow = Hp + (hl + 1) * kPS + 1;
  uint32_t diag = __shfl_up_sync(0xffffffffu, left, 1, 16);
  if (hl == 0) diag = on ? Hp[1] : 0u;
  if (shear) diag = corner;
  uint32_t last = left, fprev = 0;
  const bool top = hl == 0;
#pragma unroll 4
  for (int s = 0; s < kSlab + 15; ++s) {
    const int c = s - hl + 1;
    const uint32_t from = __shfl_up_sync(0xffffffffu, last, 1, 16);
    const bool in = (unsigned)(c - 1) < (unsigned)kSlab;
    const uint32_t up = top ? Hp[c + 1] : (shear ? fprev : from);
    fprev = from;
    const uint32_t sg = prmt((uint32_t)lds_s8(sLa + lds_u8(bL + c)), (uint32_t)lds_s8(sHa + lds_u8(bH + c)), 0xC480u);
    const uint32_t h = __viaddmax_s16x2_relu(diag, sg, __vadd2(__vmaxs2(up, left), NEG_G2));
    if (in) hrow[c] = h;
    diag = in ? up : diag;
    left = in ? h : left;
    last = in ? h : last;
  }
  __syncwarp();
}

__global__ void __launch_bounds__(128) k_sw16_tb2(Sw16Args A, int64_t first, int64_t count, uint8_t* out,
                                                   int64_t stride, int32_t* out_len, int32_t* coords, int seq_bytes) {
  extern __shared__ __align__(16) uint8_t tsm[];
  __shared__ int8_t sig_s[32 * 32];  // row stride 32, kDead outside the alphabet
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  for (int q = threadIdx.x; q < 32 * 32; q += blockDim.x) {
    const int x = q >> 5, y = q & 31;
    sig_s[q] = (x < A.asz && y < A.asz) ? A.sigma[x * A.asz + y] : (int8_t)kDead;
  }
  __syncthreads();
  const uint32_t sig32 = (uint32_t)__cvta_generic_to_shared(sig_s);
  const int half = lane >> 4, hl = lane & 15;
  const int64_t g0 = first >> 1;
  const int64_t grp = g0 + (int64_t)blockIdx.x * 4 + warp;
  const int64_t p = 2 * grp + half;
  const bool mine = p >= first && p < first + count;  // this half's problem is requested
  if (2 * grp >= first + count) return;                  // warp-uniform
  const int64_t qidx = p - first;
  PackedView V;
  V.A = &A; V.grp = grp; V.half = half;
  V.la = mine ? (int)(A.a_off[p + 1] - A.a_off[p]) : 0;
  V.lb = mine ? (int)(A.b_off[p + 1] - A.b_off[p]) : 0;
  const int la = V.la, lb = V.lb, asz = A.asz, g = A.gap;
  uint8_t* wsm = tsm + (size_t)warp * (2 * (kPW * 4 + 2 * seq_bytes));
  uint32_t* Hp = reinterpret_cast<uint32_t*>(wsm) + half * kPW;  // the halves start 16 words apart mod 32
  uint8_t* a = wsm + 2 * kPW * 4 + half * 2 * seq_bytes;
  uint8_t* ops = a + seq_bytes;  // the path, end -> start, staged in shared memory
  uint8_t* b = a + ((la + 15) & ~15) + kBPadLo;
  for (int q = hl; q < la; q += 16) a[q] = A.a_cat[A.a_off[p] + q];
  for (int q = hl - kBPadLo; q < lb + kBPadHi; q += 16) b[q] = (q >= 0 && q < lb) ? A.b_cat[A.b_off[p] + q] : kDeadCode;
  __syncwarp();
  const int best = mine ? A.scores[p] : 0;
  bool active = mine && best > 0 && la > 0 && lb > 0;
  uint8_t* o = out + (mine ? qidx : 0) * stride;
  const int ops_cap = seq_bytes;
  // 1) first lane band (row-major) whose slab maxima reach the best value (per half)
  int band8 = -1;
  const int strips = (max(la, 1) + kStrip - 1) / kStrip;
  const int nsl = (max(lb, 1) + 31 + kSlab - 1) / kSlab;  // slabs holding this problem's columns
  const int strips_w = max(__shfl_sync(0xffffffffu, strips, 0), __shfl_sync(0xffffffffu, strips, 16));
  for (int st = 0; st < strips_w; ++st) {
    for (int l2 = 0; l2 < 2; ++l2) {  // the half's 16 lanes cover the 32 lane bands in two rounds
      const int ln = hl + 16 * l2;
      bool hit = false;
      if (active && band8 < 0 && st < strips) {
        const uint32_t* sb = A.slabbest + ((grp * A.strips_max + st) * A.nslab_max) * 32 + ln;
        for (int s0 = 0; s0 < nsl; s0 += 8) {  // eight independent loads in flight
          uint32_t v[8];
#pragma unroll
          for (int q = 0; q < 8; ++q) v[q] = (s0 + q < nsl) ? __ldg(sb + (s0 + q) * 32) : 0u;
#pragma unroll
          for (int q = 0; q < 8; ++q) hit |= (s0 + q < nsl) && half16(v[q], half) + g == best;
        }
      }
      const unsigned m = __ballot_sync(0xffffffffu, hit) >> (16 * half) & 0xffffu;
      if (band8 < 0 && m) band8 = st * 32 + 16 * l2 + __ffs(m) - 1;
    }
  }
  // 2) first cell with H == best among the slabs of band8 holding the best (both halves together)
  const int lane8 = band8 >= 0 ? band8 % 32 : 0, st8 = band8 >= 0 ? band8 / 32 : 0;
  const int blk = (st8 * kStrip + lane8 * kRows) / kBlk;
  const int L0b = lane8 & ~3;
  int myr = 1 << 30, myc = 1 << 30;  // my best (row, col) candidate inside the block, row-major
  const int nsl_w = max(__shfl_sync(0xffffffffu, nsl, 0), __shfl_sync(0xffffffffu, nsl, 16));
  for (int sl = 0; sl < nsl_w; ++sl) {
    const bool cand = active && sl < nsl &&
        half16(A.slabbest[((grp * A.strips_max + st8) * A.nslab_max + sl) * 32 + lane8], half) + g == best;
    if (!__any_sync(0xffffffffu, cand)) continue;
    packed_block(V, a, b, blk, sl, cand, Hp, sig32, g, hl);
    if (cand) {
      const int D = sl * kSlab - L0b;
      for (int rr = 0; rr < 2; ++rr) {  // rows hl+1 and hl+17
        const int row = hl + 1 + 16 * rr, i = blk * kBlk + row, m = (row - 1) >> 3;
        if (i > la || row > myr) continue;
        for (int c = 1; c <= kSlab; ++c) {
          const int j = D + c - m;
          if (j >= 1 && j <= lb && hp_at(Hp, rr, hl + 1, c) == best) {
            if (row < myr || (row == myr && j < myc)) { myr = row; myc = j; }
            break;
          }
        }
      }
    }
    __syncwarp();
  }
  // smallest (row, col) over the half's lanes
  for (int o2 = 8; o2 > 0; o2 >>= 1) {
    const int orr = __shfl_xor_sync(0xffffffffu, myr, o2, 16), occ = __shfl_xor_sync(0xffffffffu, myc, o2, 16);
    if (orr < myr || (orr == myr && occ < myc)) { myr = orr; myc = occ; }
  }
  if (myr == (1 << 30)) active = false;  // cannot happen: the slab maxima name a cell holding the best
  const int ei = active ? blk * kBlk + myr : 0, ej = active ? myc : 0;
  // 3) walk back block by block; the two halves walk concurrently (leaders hl == 0)
  int i = ei, j = ej, h = active ? best : 0;
  int n = 0;
  bool overflow = false;
  while (__any_sync(0xffffffffu, h > 0)) {
    const bool on = h > 0;
    int bg = 0, sl = 0;
    if (on) {
      bg = (i - 1) / kBlk;
      const int ln = ((i - 1) % kStrip) / kRows;  // forward lane of row i
      sl = (j + ln - 1) / kSlab;
    }
    packed_block(V, a, b, bg, sl, on, Hp, sig32, g, hl);
    if (hl == 0 && on) {
      // walk in the block's sheared coordinates: packed row t (1..16) of half hf, column c
      const int R0 = bg * kBlk, D = sl * kSlab - (R0 % kStrip) / kRows;
      const int ri = i - R0;
      int hf = ri > 16 ? 1 : 0, t = ri - 16 * hf;
      int c = j - D + ((ri - 1) >> 3);
      int sh = 16 * hf;
      while (h > 0 && t >= 1 && c >= 1) {
        // branch-free step: all three neighbours are read, the move is selected
        const int tm = t - 1, cu = c - (t == 9 ? 1 : 0);  // row above: one column left at a forward-lane start
        const uint32_t* up_row = Hp + tm * kPS;
        const int dV = (int)(int16_t)(up_row[cu] >> sh), uV = (int)(int16_t)(up_row[cu + 1] >> sh);
        const int lV = (int)(int16_t)(Hp[t * kPS + c] >> sh);
        const int ra = a[i - 1], rb = b[j - 1];
        const int sub = sig_s[ra * 32 + rb];
        const bool isD = h == dV + sub;
        const bool isU = !isD && h == uV - g;
        const bool mvI = isD || isU;  // the row index moves
        const uint8_t op = isD ? (ra == rb ? 'M' : 'X') : (isU ? 'D' : 'I');
        h = isD ? dV : (isU ? uV : lV);
        i -= mvI ? 1 : 0;
        j -= isU ? 0 : 1;
        c = isD ? cu - 1 : (isU ? cu : c - 1);
        t = mvI ? tm : t;
        if (n < ops_cap) ops[n] = op;
        ++n;
        if (t == 0 && hf == 1) { hf = 0; sh = 0; t = 16; --c; }  // row 16: continue in the low half (shear 1)
      }
    }
    i = __shfl_sync(0xffffffffu, i, 16 * half);
    j = __shfl_sync(0xffffffffu, j, 16 * half);
    h = __shfl_sync(0xffffffffu, h, 16 * half);
  }
  // path start -> end, written by the half's 16 lanes
  n = __shfl_sync(0xffffffffu, n, 16 * half);
  overflow = n > stride || n > ops_cap;
  __syncwarp();
  if (mine && !overflow)
    for (int64_t u = hl; u < n; u += 16) o[u] = ops[n - 1 - u];
  if (hl == 0 && mine) {
    out_len[qidx] = overflow ? -1 : (int32_t)n;
    if (coords) {
      coords[4 * qidx] = active ? i : 0; coords[4 * qidx + 1] = active ? j : 0;
      coords[4 * qidx + 2] = ei; coords[4 * qidx + 3] = ej;
    }
  }
}

}  // namespace

bool sw16_eligible(int64_t max_la, int64_t max_lb, const int8_t* sigma_host, int asz, int gap) {
  int smax = 0, smin = 0;
  for (int q = 0; q < asz * asz; ++q) { smax = max(smax, (int)sigma_host[q]); smin = min(smin, (int)sigma_host[q]); }
  const int64_t bound = (int64_t)smax * (max_la < max_lb ? max_la : max_lb) + gap;
  return asz < 32 && bound < 32000 && smax <= 127 && smin >= -99 && gap >= 1 && gap < 1000 && (asz + 1) * kStrip <= 65535;
}

int sw16_smem_per_warp(int asz, int64_t max_la, int64_t max_lb) {
  const int prof_bytes = (asz + 1) * kStrip;
  const int64_t rec = (max_lb + 2 * kPad) * (max_la > kStrip ? rec_bytes<true>() : rec_bytes<false>());
  return (int)((2 * prof_bytes + rec + 15) & ~15);
}

void sw16_state_words(int64_t n, int64_t max_la, int64_t max_lb, int64_t* strips, int64_t* nslab, int64_t* rowck,
                      int64_t* colck, int64_t* slabbest) {
  *strips = (max_la + kStrip - 1) / kStrip;
  *nslab = (max_lb + 31 + kSlab - 1) / kSlab;  // sweep steps lbm + 31 in blocks of 32
  const int64_t groups = (n + 1) / 2;
  *rowck = groups * *strips * kBandsPerStrip * max_lb;
  *colck = groups * *strips * *nslab * kStrip;
  *slabbest = 2 * groups * *strips * *nslab * 32;  // slab maxima, then corners
}

cudaError_t sw16_solve(const Sw16Args& A, bool tb, cudaStream_t s, int64_t* launches) {
  if (A.n == 0) return cudaSuccess;
  const size_t smem = ((A.asz * A.asz + 15) & ~15) + (size_t)kWarps * A.smem_per_warp;
  const bool multi = A.max_la > kStrip;
  auto kern = tb ? (multi ? k_sw16<true, true> : k_sw16<true, false>) : (multi ? k_sw16<false, true> : k_sw16<false, false>);
  cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  // two CTAs per SM need the largest carveout
  e = cudaFuncSetAttribute(kern, cudaFuncAttributePreferredSharedMemoryCarveout, 100);
  if (e != cudaSuccess) return e;
  const int64_t groups = (A.n + 1) / 2;
  ++*launches;
  kern<<<(unsigned)((groups + kWarps - 1) / kWarps), kWarps * 32, smem, s>>>(A);
  return cudaGetLastError();
}

cudaError_t sw16_traceback(const Sw16Args& A, int64_t first, int64_t count, uint8_t* out, int64_t stride,
                           int32_t* out_len, int32_t* coords, cudaStream_t s, int64_t* launches) {
  if (count == 0) return cudaSuccess;
  const int seq_bytes = (int)(((A.max_la + 15) & ~15) + ((A.max_lb + 15) & ~15) + kBPadLo + kBPadHi);
  ++*launches;
  const size_t smem = 4 * (2 * ((size_t)kPW * 4 + 2 * (size_t)seq_bytes));
  cudaError_t e = cudaFuncSetAttribute(k_sw16_tb2, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  e = cudaFuncSetAttribute(k_sw16_tb2, cudaFuncAttributePreferredSharedMemoryCarveout, 100);
  if (e != cudaSuccess) return e;
  const int64_t groups = ((first + count - 1) >> 1) - (first >> 1) + 1;
  k_sw16_tb2<<<(unsigned)((groups + 3) / 4), 128, smem, s>>>(A, first, count, out, stride, out_len, coords,
                                                             seq_bytes);
  return cudaGetLastError();
}

}  // namespace dpk
