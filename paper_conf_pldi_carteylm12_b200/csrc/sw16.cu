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
// The column loop is split into ramp-up / steady / ramp-down so the steady
// state (all lanes inside the table) carries no bounds checks.
//
// Traceback retention without per-cell direction codes: the forward pass
// stores checkpoints of G — the bottom row of every 16-row band (odd lanes,
// every column) and every 32nd column (all rows) — plus each lane's best per
// 32-column slab (0.25 B/cell, coalesced). k_sw16_tb then recomputes only the
// 32x32 blocks the canonical traceback needs (one row per lane, the two
// 16-row halves in parallel) and walks them with the oracle's tie-break
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
constexpr int kHS = kSlab + 2;        // row stride of the recomputed block (conflict-free anti-diagonals)
// word index of H(row, col) in a recomputed block: rows 17..32 (the lower 16-row half)
// are shifted by 16 words so the two halves, which run the same anti-diagonal
// concurrently, hit disjoint banks
__device__ __forceinline__ int hbi(int row, int col) { return row * kHS + col + (row > kBand ? 16 : 0); }
constexpr int kHbWords = (kBlk + 1) * kHS + 16;
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
  uint32_t prev, last, bbest;
};

// One step of the sweep for one lane (CHECK: ramp steps where j may lie outside 1..lbm).
template <bool TB, bool CHECK>
__device__ __forceinline__ void sw_step(FwdState& S, int j, int lbm, int lane, uint32_t NEG_G2, const uint32_t* bnd,
                                        bool lane0_from_bnd, const uint16_t* offA, const uint16_t* offB,
                                        const uint8_t* profA, const uint8_t* profB, uint32_t* rowck_p,
                                        uint32_t* colck_p, uint32_t* slabbest_p) {
  const uint32_t from_above = __shfl_up_sync(0xffffffffu, S.last, 1);
  uint32_t Gu = from_above;
  if (lane == 0) Gu = (lane0_from_bnd && (!CHECK || (j >= 1 && j <= lbm))) ? bnd[j] : NEG_G2;
  const uint32_t Gd = S.prev;
  S.prev = Gu;
  if (CHECK && !(j >= 1 && j <= lbm)) return;
  // profile words of this column (residue offsets are pre-multiplied and padded with dead columns)
  const uint2 ca = *reinterpret_cast<const uint2*>(profA + offA[j + kPad - 1]);
  const uint2 cb = *reinterpret_cast<const uint2*>(profB + offB[j + kPad - 1]);
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
  S.last = g;
  if (TB) {
    if ((lane & (kLanesPerBand - 1)) == kLanesPerBand - 1) rowck_p[j - 1] = g;  // bottom row of a 16-row band
    if ((j & (kSlab - 1)) == 0 || j == lbm) {
      const int sl = (j - 1) / kSlab;
      if ((j & (kSlab - 1)) == 0) {
        uint4* col = reinterpret_cast<uint4*>(colck_p + (int64_t)(j / kSlab - 1) * kStrip);
        col[0] = make_uint4(S.G[0], S.G[1], S.G[2], S.G[3]);
        col[1] = make_uint4(S.G[4], S.G[5], S.G[6], S.G[7]);
      }
      slabbest_p[sl * 32] = S.bbest;
    }
  }
}

template <bool TB>
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
  const int offw = (int)((A.max_lb + 2 * kPad + 7) & ~7);
  uint16_t* offA = reinterpret_cast<uint16_t*>(wbase + 2 * prof_bytes);
  uint16_t* offB = offA + offw;
  uint32_t* bnd = reinterpret_cast<uint32_t*>(offB + offw);

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
  // byte offsets of each column's profile row; dead code `asz` outside each
  // problem and in the kPad columns on either side
  for (int q = lane; q < lbm + 2 * kPad; q += 32) {
    const int jj = q - kPad;  // 0-based column
    const int cA = (jj >= 0 && jj < lbA && laA > 0) ? bA[jj] : asz;
    const int cB = (jj >= 0 && jj < lbB && laB > 0) ? bB[jj] : asz;
    offA[q] = (uint16_t)(cA * kStrip);
    offB[q] = (uint16_t)(cB * kStrip);
  }
  const uint32_t NEG_G2 = (uint32_t)(uint16_t)(-gap) * 0x10001u;
  const int strips = (lam + kStrip - 1) / kStrip;
  uint32_t best2 = NEG_G2;  // max G = max h - g

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
    FwdState S;
#pragma unroll
    for (int r = 0; r < kRows; ++r) S.G[r] = NEG_G2;  // column 0: H = 0
    S.prev = NEG_G2; S.last = NEG_G2; S.bbest = NEG_G2;
    const bool from_bnd = st > 0;
    uint32_t *rowck_p = nullptr, *colck_p = nullptr, *slab_p = nullptr;
    if (TB) {
      rowck_p = A.rowck + ((grp * A.strips_max + st) * kBandsPerStrip + lane / kLanesPerBand) * A.max_lb;
      colck_p = A.colck + ((grp * A.strips_max + st) * A.nslab_max) * kStrip + lane * kRows;
      slab_p = A.slabbest + ((grp * A.strips_max + st) * A.nslab_max) * 32 + lane;
    }
    const uint8_t* pA8 = profA + lane * kRows;
    const uint8_t* pB8 = profB + lane * kRows;
    const bool spill = st + 1 < strips;
    // ramp-up (lanes above start first), steady state (every lane inside the table), ramp-down
    const int k_steady0 = 31, k_steady1 = max(31, lbm);
    int k = 0;
    for (; k < k_steady0; ++k) {
      const int j = k - lane + 1;
      sw_step<TB, true>(S, j, lbm, lane, NEG_G2, bnd, from_bnd, offA, offB, pA8, pB8, rowck_p, colck_p, slab_p);
      if (j >= 1 && j <= lbm) {
        if (spill && lane == 31) bnd[j] = S.last;
        if ((j & (kSlab - 1)) == 0) { best2 = __vmaxs2(best2, S.bbest); S.bbest = NEG_G2; }
      }
      __syncwarp();
    }
#pragma unroll 2
    for (; k < k_steady1; ++k) {
      const int j = k - lane + 1;
      sw_step<TB, false>(S, j, lbm, lane, NEG_G2, bnd, from_bnd, offA, offB, pA8, pB8, rowck_p, colck_p, slab_p);
      if (spill && lane == 31) bnd[j] = S.last;
      if ((j & (kSlab - 1)) == 0) { best2 = __vmaxs2(best2, S.bbest); S.bbest = NEG_G2; }
      __syncwarp();
    }
    for (; k < lbm + 31; ++k) {
      const int j = k - lane + 1;
      sw_step<TB, true>(S, j, lbm, lane, NEG_G2, bnd, from_bnd, offA, offB, pA8, pB8, rowck_p, colck_p, slab_p);
      if (j >= 1 && j <= lbm) {
        if (spill && lane == 31) bnd[j] = S.last;
        if ((j & (kSlab - 1)) == 0) { best2 = __vmaxs2(best2, S.bbest); S.bbest = NEG_G2; }
      }
      __syncwarp();
    }
    best2 = __vmaxs2(best2, S.bbest);
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) best2 = __vmaxs2(best2, __shfl_xor_sync(0xffffffffu, best2, o));
  if (lane == 0) {
    A.scores[pA] = lo16(best2) + gap;
    if (hasB) A.scores[pB] = hi16(best2) + gap;
  }
}

// ---------------------------------------------------------------- traceback
struct TbView {
  const Sw16Args* A;
  int64_t grp;
  int half;
  int la, lb;
  // H at row 32*band (the bottom row of band-1), column j; 0 on the borders
  __device__ __forceinline__ int top_h(int band, int j) const {
    if (band == 0 || j == 0) return 0;
    const int b = band - 1;
    const int st = b / kBandsPerStrip, bi = b % kBandsPerStrip;
    const uint32_t v = A->rowck[((grp * A->strips_max + st) * kBandsPerStrip + bi) * A->max_lb + (j - 1)];
    return half16(v, half) + A->gap;
  }
  // H at row i (1-based), column 32*slab
  __device__ __forceinline__ int left_h(int i, int slab) const {
    if (slab == 0) return 0;
    const int st = (i - 1) / kStrip, ri = (i - 1) % kStrip;
    const uint32_t v = A->colck[((grp * A->strips_max + st) * A->nslab_max + (slab - 1)) * kStrip + ri];
    return half16(v, half) + A->gap;
  }
};

// Recompute the 32-row block `blk` x slab into Hb[(r+1)*kHS + c] (row 0 / column 0 =
// boundaries); one row per lane. The two 16-row halves are independent given the
// checkpoint row between them, so lanes 0-15 and 16-31 run concurrently (47 steps).
__device__ void recompute_block(const TbView& V, const uint8_t* a, const uint8_t* b, int blk, int slab, int* Hb,
                                int* mid, const int8_t* sig_s, int asz, int g) {
  const int lane = threadIdx.x & 31;
  const int R0 = blk * kBlk, C0 = slab * kSlab;
  const int band0 = R0 / kBand;
  for (int c = lane; c <= kSlab; c += 32) {
    Hb[c] = (C0 + c <= V.lb) ? V.top_h(band0, C0 + c) : 0;
    mid[c] = (C0 + c <= V.lb) ? V.top_h(band0 + 1, C0 + c) : 0;
  }
  const int i = R0 + lane + 1;
  const bool row_ok = i <= V.la;
  int left = row_ok ? V.left_h(i, slab) : 0;
  Hb[hbi(lane + 1, 0)] = left;
  __syncwarp();
  const int hl = lane & (kBand - 1);  // row within the half
  const int* top = (lane < kBand) ? Hb : mid;
  const int ai = row_ok ? a[i - 1] : 0;
  const int8_t* srow = sig_s + ai * asz;
  const uint8_t* bb = b + C0 - 1;      // bb[c] = b[C0 + c - 1]
  const int cmax = min(kSlab, V.lb - C0);  // live columns of this slab
  int* hrow = Hb + hbi(lane + 1, 0);
  int diag = __shfl_up_sync(0xffffffffu, left, 1);
  if (hl == 0) diag = top[0];
  int last = 0;
  // branch-free wavefront: every lane evaluates every step, out-of-range steps are masked
#pragma unroll 4
  for (int s = 0; s < kSlab + kBand - 1; ++s) {
    const int c = s - hl + 1;
    const int from = __shfl_up_sync(0xffffffffu, last, 1);
    const bool in = (unsigned)(c - 1) < (unsigned)kSlab;
    const int cc = in ? c : 1;
    const int up = (hl == 0) ? top[cc] : from;
    int h = max(max(diag + srow[cc <= cmax ? bb[cc] : 0], 0), max(up, left) - g);
    h = (row_ok && cc <= cmax) ? h : 0;
    if (in) hrow[cc] = h;
    diag = in ? up : diag;
    left = in ? h : left;
    last = in ? h : last;
  }
  __syncwarp();
}

__global__ void __launch_bounds__(128) k_sw16_tb(Sw16Args A, int64_t first, int64_t count, uint8_t* out,
                                                  int64_t stride, int32_t* out_len, int32_t* coords, int seq_bytes) {
  extern __shared__ __align__(16) uint8_t tsm[];
  __shared__ int8_t sig_s[32 * 32];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  for (int q = threadIdx.x; q < A.asz * A.asz; q += blockDim.x) sig_s[q] = A.sigma[q];
  __syncthreads();
  const int64_t qidx = (int64_t)blockIdx.x * 4 + warp;
  if (qidx >= count) return;
  const int64_t p = first + qidx;
  TbView V;
  V.A = &A;
  V.grp = p >> 1;
  V.half = (int)(p & 1);
  uint8_t* wsm = tsm + (size_t)warp * (seq_bytes + (kHbWords + kHS) * 4);
  int* Hb = reinterpret_cast<int*>(wsm);
  int* mid = Hb + kHbWords;
  uint8_t* a = wsm + (kHbWords + kHS) * 4;
  V.la = (int)(A.a_off[p + 1] - A.a_off[p]);
  V.lb = (int)(A.b_off[p + 1] - A.b_off[p]);
  const int la = V.la, lb = V.lb, asz = A.asz, g = A.gap;
  uint8_t* b = a + ((la + 15) & ~15);
  // stage both sequences in shared memory: the walk and the block recomputes read them per cell
  for (int q = lane; q < la; q += 32) a[q] = A.a_cat[A.a_off[p] + q];
  for (int q = lane; q < lb; q += 32) b[q] = A.b_cat[A.b_off[p] + q];
  __syncwarp();
  const int best = A.scores[p];
  uint8_t* o = out + qidx * stride;
  if (best <= 0 || la == 0 || lb == 0) {
    if (lane == 0) {
      out_len[qidx] = 0;
      if (coords) { coords[4 * qidx] = 0; coords[4 * qidx + 1] = 0; coords[4 * qidx + 2] = 0; coords[4 * qidx + 3] = 0; }
    }
    return;
  }
  // 1) first lane band (row-major order) whose slab maxima reach the best value
  const int strips = (la + kStrip - 1) / kStrip;
  const int nsl = (lb + kSlab - 1) / kSlab;
  int band8 = -1;
  for (int st = 0; st < strips && band8 < 0; ++st) {
    bool hit = false;
    for (int sl = 0; sl < nsl; ++sl) {
      const uint32_t v = A.slabbest[((V.grp * A.strips_max + st) * A.nslab_max + sl) * 32 + lane];
      hit |= half16(v, V.half) + g == best;
    }
    const unsigned m = __ballot_sync(0xffffffffu, hit);
    if (m) band8 = st * 32 + __ffs(m) - 1;
  }
  const int lane8 = band8 % 32, st8 = band8 / 32;
  // 2) first cell with H == best: recompute only the slabs of band8 holding the best,
  //    within the 32-row block that contains band8's rows
  const int band = (st8 * kStrip + lane8 * kRows) / kBlk;
  int myc = 1 << 30;
  for (int sl = 0; sl < nsl; ++sl) {
    const uint32_t v = A.slabbest[((V.grp * A.strips_max + st8) * A.nslab_max + sl) * 32 + lane8];
    if (half16(v, V.half) + g != best) continue;
    recompute_block(V, a, b, band, sl, Hb, mid, sig_s, asz, g);
    const int i = band * kBlk + lane + 1;
    if (myc == (1 << 30) && i <= la)
      for (int c = 1; c <= kSlab; ++c) {
        const int j = sl * kSlab + c;
        if (j <= lb && Hb[hbi(lane + 1, c)] == best) { myc = j; break; }
      }
    __syncwarp();
  }
  const unsigned hm = __ballot_sync(0xffffffffu, myc != (1 << 30));
  const int rowl = __ffs(hm) - 1;
  const int ej = __shfl_sync(0xffffffffu, myc, rowl < 0 ? 0 : rowl);
  const int ei = band * kBlk + rowl + 1;
  // 3) walk back block by block
  int i = ei, j = ej, h = best;
  int64_t n = 0;
  bool overflow = false;
  while (h > 0) {
    const int bg = (i - 1) / kBlk, sl = (j - 1) / kSlab;
    recompute_block(V, a, b, bg, sl, Hb, mid, sig_s, asz, g);
    if (lane == 0) {
      const int R0 = bg * kBlk, C0 = sl * kSlab;
      while (h > 0 && i > R0 && j > C0) {
        const int ri = i - R0, cj = j - C0;
        const int sub = sig_s[a[i - 1] * asz + b[j - 1]];
        uint8_t op;
        if (h == Hb[hbi(ri - 1, cj - 1)] + sub) {
          op = (a[i - 1] == b[j - 1]) ? 'M' : 'X';
          --i; --j;
        } else if (h == Hb[hbi(ri - 1, cj)] - g) {
          op = 'D'; --i;
        } else {
          op = 'I'; --j;
        }
        h = Hb[hbi(i - R0, j - C0)];
        if (n < stride) o[n] = op; else overflow = true;
        ++n;
      }
    }
    i = __shfl_sync(0xffffffffu, i, 0);
    j = __shfl_sync(0xffffffffu, j, 0);
    h = __shfl_sync(0xffffffffu, h, 0);
  }
  if (lane == 0) {
    if (!overflow)
      for (int64_t u = 0, v = n - 1; u < v; ++u, --v) { const uint8_t t = o[u]; o[u] = o[v]; o[v] = t; }
    out_len[qidx] = overflow ? -1 : (int32_t)n;
    if (coords) { coords[4 * qidx] = i; coords[4 * qidx + 1] = j; coords[4 * qidx + 2] = ei; coords[4 * qidx + 3] = ej; }
  }
}

// ---------------------------------------------------------------- packed traceback
// Two problems per warp (the pair group of the forward pass): lanes 0-15 serve
// problem 2g, lanes 16-31 problem 2g+1. A 32-row block is recomputed by 16 lanes,
// lane hl holding rows hl+1 (low half) and hl+17 (high half) in one s16x2
// register — the two 16-row halves are independent given the checkpoint row
// between them — so one VIADDMNMX.S16x2 chain step evaluates two cells.
// Hp[t][c] packs (H(R0+t, C0+c), H(R0+16+t, C0+c)), t = 0..16: row 0 holds the
// checkpoint rows (top, middle), column 0 the checkpoint column.
constexpr int kPS = kSlab + 2;        // packed row stride (words)
constexpr int kPW = 17 * kPS + 14;    // words per packed block (592 = 16 mod 32: the halves hit disjoint banks)

struct PackedView {
  const Sw16Args* A;
  int64_t grp;
  int half, la, lb;
  __device__ __forceinline__ int top_h(int band, int j) const {  // H at row 16*band, column j
    if (band == 0 || j == 0) return 0;
    const int b = band - 1;
    const int st = b / kBandsPerStrip, bi = b % kBandsPerStrip;
    const uint32_t v = A->rowck[((grp * A->strips_max + st) * kBandsPerStrip + bi) * A->max_lb + (j - 1)];
    return half16(v, half) + A->gap;
  }
  __device__ __forceinline__ int left_h(int i, int slab) const {  // H at row i, column 32*slab
    if (slab == 0) return 0;
    const int st = (i - 1) / kStrip, ri = (i - 1) % kStrip;
    const uint32_t v = A->colck[((grp * A->strips_max + st) * A->nslab_max + (slab - 1)) * kStrip + ri];
    return half16(v, half) + A->gap;
  }
};

__device__ __forceinline__ uint32_t pk(int lo, int hi) { return (uint32_t)(uint16_t)lo | ((uint32_t)(uint16_t)hi << 16); }
__device__ __forceinline__ int hp_get(const uint32_t* Hp, int row, int col) {  // H(R0 + row, C0 + col), row 0..32
  return row <= 16 ? lo16(Hp[row * kPS + col]) : hi16(Hp[(row - 16) * kPS + col]);
}

// Recompute this half's block (blk, slab) into Hp; `on` = this half has a block to do.
__device__ void packed_block(const PackedView& V, const uint8_t* a, const uint8_t* b, int blk, int slab, bool on,
                             uint32_t* Hp, const int8_t* sig_s, int asz, int g, int hl) {
  const int R0 = blk * kBlk, C0 = slab * kSlab;
  const int band0 = R0 / kBand;
  if (on) {
    for (int c = hl; c <= kSlab; c += 16)
      Hp[c] = (C0 + c <= V.lb) ? pk(V.top_h(band0, C0 + c), V.top_h(band0 + 1, C0 + c)) : 0u;
  }
  const int iL = R0 + hl + 1, iH = R0 + hl + 17;
  const bool okL = on && iL <= V.la, okH = on && iH <= V.la;
  uint32_t left = pk(okL ? V.left_h(iL, slab) : 0, okH ? V.left_h(iH, slab) : 0);
  if (on) Hp[(hl + 1) * kPS] = left;
  __syncwarp();
  const int8_t* sL = sig_s + (okL ? a[iL - 1] : 0) * asz;
  const int8_t* sH = sig_s + (okH ? a[iH - 1] : 0) * asz;
  const uint32_t rowmask = (okL ? 0xffffu : 0u) | (okH ? 0xffff0000u : 0u);
  const uint8_t* bb = b + C0 - 1;
  const int cmax = on ? min(kSlab, V.lb - C0) : 0;
  const uint32_t NEG_G2 = (uint32_t)(uint16_t)(-g) * 0x10001u;
  uint32_t* hrow = Hp + (hl + 1) * kPS;
  uint32_t diag = __shfl_up_sync(0xffffffffu, left, 1, 16);
  if (hl == 0) diag = on ? Hp[0] : 0u;
  uint32_t last = 0;
#pragma unroll 4
  for (int s = 0; s < kSlab + 15; ++s) {
    const int c = s - hl + 1;
    const uint32_t from = __shfl_up_sync(0xffffffffu, last, 1, 16);
    const bool in = (unsigned)(c - 1) < (unsigned)kSlab;
    const int cc = in ? c : 1;
    const uint32_t up = (hl == 0) ? Hp[cc] : from;
    const int bj = (cc <= cmax) ? bb[cc] : 0;  // never read past the staged sequence
    const uint32_t sg = prmt((uint32_t)(uint8_t)sL[bj], (uint32_t)(uint8_t)sH[bj], 0xC480u);
    uint32_t h = __viaddmax_s16x2_relu(diag, sg, __vadd2(__vmaxs2(up, left), NEG_G2));
    h = (cc <= cmax) ? (h & rowmask) : 0u;
    if (in) hrow[cc] = h;
    diag = in ? up : diag;
    left = in ? h : left;
    last = in ? h : last;
  }
  __syncwarp();
}

__global__ void __launch_bounds__(128) k_sw16_tb2(Sw16Args A, int64_t first, int64_t count, uint8_t* out,
                                                   int64_t stride, int32_t* out_len, int32_t* coords, int seq_bytes) {
  extern __shared__ __align__(16) uint8_t tsm[];
  __shared__ int8_t sig_s[32 * 32];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  for (int q = threadIdx.x; q < A.asz * A.asz; q += blockDim.x) sig_s[q] = A.sigma[q];
  __syncthreads();
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
  uint8_t* b = a + ((la + 15) & ~15);
  for (int q = hl; q < la; q += 16) a[q] = A.a_cat[A.a_off[p] + q];
  for (int q = hl; q < lb; q += 16) b[q] = A.b_cat[A.b_off[p] + q];
  __syncwarp();
  const int best = mine ? A.scores[p] : 0;
  bool active = mine && best > 0 && la > 0 && lb > 0;
  uint8_t* o = out + (mine ? qidx : 0) * stride;
  const int ops_cap = seq_bytes;
  // 1) first lane band (row-major) whose slab maxima reach the best value (per half)
  int band8 = -1;
  const int strips = (max(la, 1) + kStrip - 1) / kStrip;
  const int nsl = (max(lb, 1) + kSlab - 1) / kSlab;
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
  int myr = 1 << 30, myc = 1 << 30;  // my best (row, col) candidate inside the block, row-major
  const int nsl_w = max(__shfl_sync(0xffffffffu, nsl, 0), __shfl_sync(0xffffffffu, nsl, 16));
  for (int sl = 0; sl < nsl_w; ++sl) {
    const bool cand = active && sl < nsl &&
        half16(A.slabbest[((grp * A.strips_max + st8) * A.nslab_max + sl) * 32 + lane8], half) + g == best;
    if (!__any_sync(0xffffffffu, cand)) continue;
    packed_block(V, a, b, blk, sl, cand, Hp, sig_s, asz, g, hl);
    if (cand) {
      for (int rr = 0; rr < 2; ++rr) {  // rows hl+1 and hl+17
        const int row = hl + 1 + 16 * rr, i = blk * kBlk + row;
        if (i > la || row > myr) continue;
        for (int c = 1; c <= kSlab; ++c) {
          const int j = sl * kSlab + c;
          if (j <= lb && hp_get(Hp, row, c) == best) {
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
  int64_t n = 0;
  bool overflow = false;
  while (__any_sync(0xffffffffu, h > 0)) {
    const bool on = h > 0;
    const int bg = on ? (i - 1) / kBlk : 0, sl = on ? (j - 1) / kSlab : 0;
    packed_block(V, a, b, bg, sl, on, Hp, sig_s, asz, g, hl);
    if (hl == 0 && on) {
      const int R0 = bg * kBlk, C0 = sl * kSlab;
      while (h > 0 && i > R0 && j > C0) {
        const int ri = i - R0, cj = j - C0;
        const int sub = sig_s[a[i - 1] * asz + b[j - 1]];
        uint8_t op;
        if (h == hp_get(Hp, ri - 1, cj - 1) + sub) {
          op = (a[i - 1] == b[j - 1]) ? 'M' : 'X';
          --i; --j;
        } else if (h == hp_get(Hp, ri - 1, cj) - g) {
          op = 'D'; --i;
        } else {
          op = 'I'; --j;
        }
        h = hp_get(Hp, i - R0, j - C0);
        if (n < ops_cap) ops[n] = op;
        ++n;
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
  return asz <= 32 && bound < 32000 && smax <= 127 && smin >= -99 && gap < 1000 && (asz + 1) * kStrip <= 65535;
}

int sw16_smem_per_warp(int asz, int64_t max_la, int64_t max_lb) {
  const int prof_bytes = (asz + 1) * kStrip;
  const int64_t offw = (max_lb + 2 * kPad + 7) & ~int64_t(7);
  const int64_t bnd = (max_la > kStrip) ? 4 * (max_lb + 1) : 0;  // boundary row only for multi-strip
  return (int)((2 * prof_bytes + 2 * 2 * offw + bnd + 15) & ~15);
}

void sw16_state_words(int64_t n, int64_t max_la, int64_t max_lb, int64_t* strips, int64_t* nslab, int64_t* rowck,
                      int64_t* colck, int64_t* slabbest) {
  *strips = (max_la + kStrip - 1) / kStrip;
  *nslab = (max_lb + kSlab - 1) / kSlab;
  if (*nslab < 1) *nslab = 1;
  const int64_t groups = (n + 1) / 2;
  *rowck = groups * *strips * kBandsPerStrip * max_lb;
  *colck = groups * *strips * *nslab * kStrip;
  *slabbest = groups * *strips * *nslab * 32;
}

cudaError_t sw16_solve(const Sw16Args& A, bool tb, cudaStream_t s, int64_t* launches) {
  if (A.n == 0) return cudaSuccess;
  const size_t smem = ((A.asz * A.asz + 15) & ~15) + (size_t)kWarps * A.smem_per_warp;
  auto kern = tb ? k_sw16<true> : k_sw16<false>;
  cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  const int64_t groups = (A.n + 1) / 2;
  ++*launches;
  kern<<<(unsigned)((groups + kWarps - 1) / kWarps), kWarps * 32, smem, s>>>(A);
  return cudaGetLastError();
}

cudaError_t sw16_traceback(const Sw16Args& A, int64_t first, int64_t count, uint8_t* out, int64_t stride,
                           int32_t* out_len, int32_t* coords, cudaStream_t s, int64_t* launches) {
  if (count == 0) return cudaSuccess;
  const int seq_bytes = (int)(((A.max_la + 15) & ~15) + ((A.max_lb + 15) & ~15));
  ++*launches;
  if (getenv("DP_SW_TB_UNPACKED") == nullptr) {  // packed: two problems per warp
    const size_t smem = 4 * (2 * ((size_t)kPW * 4 + 2 * (size_t)seq_bytes));
    cudaError_t e = cudaFuncSetAttribute(k_sw16_tb2, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    const int64_t groups = ((first + count - 1) >> 1) - (first >> 1) + 1;
    k_sw16_tb2<<<(unsigned)((groups + 3) / 4), 128, smem, s>>>(A, first, count, out, stride, out_len, coords,
                                                               seq_bytes);
    return cudaGetLastError();
  }
  const size_t smem = 4 * ((size_t)seq_bytes + (kHbWords + kHS) * 4);
  cudaError_t e = cudaFuncSetAttribute(k_sw16_tb, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  k_sw16_tb<<<(unsigned)((count + 3) / 4), 128, smem, s>>>(A, first, count, out, stride, out_len, coords, seq_bytes);
  return cudaGetLastError();
}

}  // namespace dpk
