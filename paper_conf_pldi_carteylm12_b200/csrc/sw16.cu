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
// (0.25 B/cell), plus every lane's maximum over the strip. k_sw16_tb3 recomputes
// only the 32x32 (sheared) blocks the canonical traceback needs and walks them
// with the oracle's tie-break (diag > up > left, stop at H = 0; end cell = first
// maximum in row-major order).
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
    uint32_t sbest = NEG_G2;  // this lane's maximum over the strip (TB)
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
        sbest = __vmaxs2(sbest, S.bbest);
        S.best2 = __vmaxs2(S.best2, S.bbest);
        S.bbest = NEG_G2;
      }
    }
    S.best2 = __vmaxs2(S.best2, S.bbest);
    if (TB) A.lanebest[(grp * A.strips_max + st) * 32 + lane] = sbest;
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
// k_sw16_tb3: one warp serves 8 forward pairs (problems 2g, 2g+1), one pair per
// 4-lane group. A traceback "block" is 32 rows (forward lanes L0..L0+3 of one
// strip, L0 = 4 (blk mod 8)) x one slab: forward lane L0+m covered columns
// j = D + c - m, c = 1..32, D = 32 slab - L0, at forward steps 32 slab + c - 1.
// So in the sheared column c all four lanes are at the SAME forward step and
// group lane m re-runs forward lane L0+m (8 rows) for 32 steps exactly as the
// sweep did (no ramp): the left column is its checkpoint, its first diagonal the
// corner word, lane 0's "up" the band checkpoint row above the block. The two
// s16x2 halves carry the pair's two problems, each with its own block. The G of
// the block go to shared memory column-major; the canonical walk (diag > up >
// left, stop at H = 0) then runs on one lane per problem, 16 walkers per warp.
// The end cell (first row-major maximum) comes from the per-lane strip maxima,
// then the slabs of that lane whose maximum equals the score.
constexpr int kCS = 36;                  // words per block column: row t (-1..31) at t + 4
constexpr int kGS = 34 * kCS + 4;        // words per group buffer (columns c = -1..32); = 4 mod 8
constexpr int kBS = 40;                  // staged b residues per half (columns D-3 .. D+32)
constexpr int kDeadCode = 31;            // residue code whose sigma row/column is kDead (alphabets < 32)
constexpr int kOpsCap = 512;             // ops staged in shared memory per problem (longer paths spill to the row tail)

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
__device__ __forceinline__ uint32_t join(uint32_t lo_src, uint32_t hi_src) { return prmt(lo_src, hi_src, 0x7610u); }
__device__ __forceinline__ void prefetch_l2(const void* p) { asm volatile("prefetch.global.L2 [%0];" ::"l"(p)); }

struct TbHalf {       // one problem of the pair (uniform within its group)
  int64_t p;          // problem id
  const uint8_t *a, *b;
  int la, lb, best;
  int mode;           // 0 done / idle, 1 end-cell search, 2 walk
  int band;           // search: first lane band (strip*32 + lane) reaching the score
  int scur, cand;     // search: next slab to probe, candidate slab (-1 none)
  long long found;    // search: row-major key (i << 32 | j) of the first maximum
  int i, j, h, n;     // walk state
  int ei, ej;         // end cell
  int blk, sl, on;    // this round's block
};

__global__ void __launch_bounds__(32) k_sw16_tb3(Sw16Args A, int64_t first, int64_t count, uint8_t* out,
                                                  int64_t stride, int32_t* out_len, int32_t* coords) {
  extern __shared__ __align__(16) uint8_t tsm[];
  int8_t* sig_s = reinterpret_cast<int8_t*>(tsm);                 // [32][32], kDead outside the alphabet
  const int lane = threadIdx.x, gq = lane >> 2, m = lane & 3;
  for (int q = lane; q < 32 * 32; q += 32) {
    const int x = q >> 5, y = q & 31;
    sig_s[q] = (x < A.asz && y < A.asz) ? A.sigma[x * A.asz + y] : (int8_t)kDead;
  }
  uint32_t* Hs = reinterpret_cast<uint32_t*>(tsm + 1024) + gq * kGS;
  uint8_t* bS = tsm + 1024 + 8 * kGS * 4 + gq * 2 * kBS;           // [2][kBS] staged b residues
  uint8_t* aS = tsm + 1024 + 8 * kGS * 4 + 8 * 2 * kBS + gq * 2 * kBlk;  // [2][32] staged a residues
  uint8_t* opsS = tsm + 1024 + 8 * kGS * 4 + 8 * 2 * kBS + 8 * 2 * kBlk + gq * 2 * kOpsCap;  // [2][cap] ops
  const uint32_t sig32 = (uint32_t)__cvta_generic_to_shared(sig_s);
  const uint32_t hs32 = (uint32_t)__cvta_generic_to_shared(Hs);
  const uint32_t bs32 = (uint32_t)__cvta_generic_to_shared(bS);
  const unsigned full = 0xffffffffu;
  const int g = A.gap;
  const uint32_t NEG_G2 = (uint32_t)(uint16_t)(-g) * 0x10001u;
  const int64_t grp = (first >> 1) + (int64_t)blockIdx.x * 8 + gq;
  const int64_t SM = A.strips_max, NS = A.nslab_max;
  PhaseClock clk;
  clk.dbg = A.dbg;
  clk.start();

  TbHalf H[2];
#pragma unroll
  for (int hf = 0; hf < 2; ++hf) {
    TbHalf& X = H[hf];
    X.p = 2 * grp + hf;
    const bool mine = X.p >= first && X.p < first + count;
    X.la = mine ? (int)(A.a_off[X.p + 1] - A.a_off[X.p]) : 0;
    X.lb = mine ? (int)(A.b_off[X.p + 1] - A.b_off[X.p]) : 0;
    X.a = mine ? A.a_cat + A.a_off[X.p] : A.a_cat;
    X.b = mine ? A.b_cat + A.b_off[X.p] : A.b_cat;
    X.best = mine ? A.scores[X.p] : 0;
    X.mode = (mine && X.best > 0 && X.la > 0 && X.lb > 0) ? 1 : 0;
    X.band = -1; X.scur = 0; X.cand = -1; X.found = -1;
    X.i = X.j = X.h = X.n = 0; X.ei = X.ej = 0;
    X.blk = X.sl = X.on = 0;
  }
  // 1) first lane band (row-major: strip, lane) whose strip maximum reaches the score
  {
    int stw = max((H[0].la + kStrip - 1) / kStrip, (H[1].la + kStrip - 1) / kStrip);
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) stw = max(stw, __shfl_xor_sync(full, stw, o));
    for (int st = 0; st < stw; ++st) {
      uint32_t w[8];
#pragma unroll
      for (int q = 0; q < 8; ++q)
        w[q] = (H[0].mode | H[1].mode) && grp < (A.n + 1) / 2 && st < SM
                   ? __ldcg(A.lanebest + (grp * SM + st) * 32 + 8 * m + q) : 0u;
#pragma unroll
      for (int hf = 0; hf < 2; ++hf) {
        TbHalf& X = H[hf];
        const bool want = X.mode == 1 && X.band < 0 && st * kStrip < X.la;
        int firstl = 32;
#pragma unroll
        for (int q = 7; q >= 0; --q)
          if (want && half16(w[q], hf) + g == X.best) firstl = 8 * m + q;
        firstl = min(firstl, __shfl_xor_sync(full, firstl, 1));
        firstl = min(firstl, __shfl_xor_sync(full, firstl, 2));
        if (want && firstl < 32) X.band = st * 32 + firstl;
      }
    }
#pragma unroll
    for (int hf = 0; hf < 2; ++hf)
      if (H[hf].mode == 1 && H[hf].band < 0) H[hf].mode = 0;  // cannot happen: the maxima name the score
  }
  __syncwarp();
  clk.lap(0);

  int guard = 8 * (int)((A.max_la + A.max_lb) / 16 + 8);
  while (__any_sync(full, (H[0].mode | H[1].mode) != 0) && --guard > 0) {
    // 2) searching halves: next candidate slab of their lane band (32 slabs per probe)
    for (;;) {
      bool need[2];
#pragma unroll
      for (int hf = 0; hf < 2; ++hf) need[hf] = H[hf].mode == 1 && H[hf].cand < 0;
      if (!__any_sync(full, need[0] || need[1])) break;
#pragma unroll
      for (int hf = 0; hf < 2; ++hf) {
        TbHalf& X = H[hf];
        const int nsl = (X.lb + 31 + kSlab - 1) / kSlab;
        const int st8 = X.band >> 5, ln8 = X.band & 31;
        uint32_t bits = 0;
        if (need[hf]) {
          const uint32_t* sb = A.slabbest + ((grp * SM + st8) * NS) * 32 + ln8;
#pragma unroll
          for (int q = 0; q < 8; ++q) {
            const int s = X.scur + m + 4 * q;
            if (s < nsl && half16(__ldcg(sb + (int64_t)s * 32), hf) + g == X.best) bits |= 1u << (m + 4 * q);
          }
        }
        bits |= __shfl_xor_sync(full, bits, 1);
        bits |= __shfl_xor_sync(full, bits, 2);
        if (need[hf]) {
          if (bits) {
            X.cand = X.scur + __ffs(bits) - 1;
          } else {
            X.scur += 32;
            if (X.scur >= nsl) {  // candidates exhausted: walk from the first maximum
              if (X.found >= 0) {
                X.mode = 2;
                X.i = X.ei = (int)(X.found >> 32);
                X.j = X.ej = (int)(X.found & 0xffffffffll);
                X.h = X.best;
              } else {
                X.mode = 0;  // cannot happen
              }
            }
          }
        }
      }
    }
    clk.lap(1);
    if (clk.dbg) clk.acc[7] += 1;
    // 3) this round's block per half
#pragma unroll
    for (int hf = 0; hf < 2; ++hf) {
      TbHalf& X = H[hf];
      X.on = 0;
      if (X.mode == 1 && X.cand >= 0) {
        const int st8 = X.band >> 5, ln8 = X.band & 31;
        X.blk = st8 * (kStrip / kBlk) + ln8 / 4;
        X.sl = X.cand;
        X.on = 1;
      } else if (X.mode == 2) {
        const int ln = ((X.i - 1) % kStrip) / kRows;
        X.blk = (X.i - 1) / kBlk;
        X.sl = (X.j + ln - 1) / kSlab;
        X.on = 1;
      }
    }
    // 3b) walking halves: the block after this one is above, above-left or left of it;
    // pull their checkpoints into L2 now so the next round's loads do not go to DRAM.
#pragma unroll
    for (int hf = 0; hf < 2; ++hf) {
      const TbHalf& X = H[hf];
      if (X.mode != 2) continue;
#pragma unroll
      for (int q = 0; q < 3; ++q) {
        const int nb = X.blk - (q < 2 ? 1 : 0), ns = X.sl - (q > 0 ? 1 : 0);
        if (nb < 0 || ns < 1) continue;
        const int r0 = nb * kBlk, st = r0 / kStrip, L0 = (r0 % kStrip) / kRows;
        const int64_t base = (grp * SM + st) * NS + (ns - 1);
        prefetch_l2(A.colck + base * kStrip + (L0 + m) * kRows);
        if (m == 0) prefetch_l2(A.corner + base * 32 + L0);
        if (r0 > 0) {
          const int bnd = r0 / kBand - 1, j0 = max(1, ns * kSlab - L0 + 16 * m);
          if (j0 <= X.lb)
            prefetch_l2(A.rowck + ((grp * SM + bnd / kBandsPerStrip) * kBandsPerStrip + bnd % kBandsPerStrip) * A.max_lb +
                        (j0 - 1));
        }
      }
    }
    // 4) recompute both blocks. Every global load of the round is issued before any
    // shared-memory store (checkpoint column, corner, a and b residues, top row).
    int R0[2], D[2];
    uint32_t sa[2][kRows];
    uint32_t Gs[kRows], prev;
    {
      uint32_t w[2][kRows], cw[2], av[2][kRows], bv[2][kBS / 4], tv[2][9];
#pragma unroll
      for (int hf = 0; hf < 2; ++hf) {
        TbHalf& X = H[hf];
        R0[hf] = X.blk * kBlk;
        const int st = R0[hf] / kStrip, L0 = (R0[hf] % kStrip) / kRows, l = L0 + m;
        D[hf] = X.sl * kSlab - L0;
        const bool ck = X.on && X.sl > 0;
        const int64_t base = (grp * SM + st) * NS + (ck ? X.sl - 1 : 0);
        const uint4* cp = reinterpret_cast<const uint4*>(A.colck + base * kStrip + l * kRows);
        const uint4 v0 = ck ? __ldcg(cp) : make_uint4(NEG_G2, NEG_G2, NEG_G2, NEG_G2);
        const uint4 v1 = ck ? __ldcg(cp + 1) : make_uint4(NEG_G2, NEG_G2, NEG_G2, NEG_G2);
        w[hf][0] = v0.x; w[hf][1] = v0.y; w[hf][2] = v0.z; w[hf][3] = v0.w;
        w[hf][4] = v1.x; w[hf][5] = v1.y; w[hf][6] = v1.z; w[hf][7] = v1.w;
        cw[hf] = ck ? __ldcg(A.corner + base * 32 + l) : NEG_G2;
#pragma unroll
        for (int r = 0; r < kRows; ++r) {
          const int i = R0[hf] + 8 * m + r + 1;
          av[hf][r] = (X.on && i <= X.la) ? __ldg(X.a + i - 1) : (uint32_t)kDeadCode;
        }
#pragma unroll
        for (int k = 0; k < kBS / 4; ++k) {  // b residues of columns D-3 .. D+36 (x = j - D + 3)
          const int j = D[hf] + m + 4 * k - 3;
          bv[hf][k] = (X.on && j >= 1 && j <= X.lb) ? __ldg(X.b + j - 1) : (uint32_t)kDeadCode;
        }
        // top row (G of row R0, columns D + c, c = 0..32): the band checkpoint above the block
        const int bnd = R0[hf] / kBand - 1;
        const uint32_t* rk = A.rowck + ((grp * SM + (bnd >= 0 ? bnd / kBandsPerStrip : 0)) * kBandsPerStrip +
                                        (bnd >= 0 ? bnd % kBandsPerStrip : 0)) * A.max_lb - 1;
#pragma unroll
        for (int k = 0; k < 9; ++k) {
          const int c = m + 4 * k, j = D[hf] + c;
          tv[hf][k] = (X.on && bnd >= 0 && c <= kSlab && j >= 1 && j <= X.lb) ? __ldcg(rk + j) : NEG_G2;
        }
      }
#pragma unroll
      for (int hf = 0; hf < 2; ++hf) {
#pragma unroll
        for (int r = 0; r < kRows; ++r) {
          sa[hf][r] = sig32 + 32 * av[hf][r];
          aS[hf * kBlk + 8 * m + r] = (uint8_t)av[hf][r];
        }
#pragma unroll
        for (int k = 0; k < kBS / 4; ++k) bS[hf * kBS + m + 4 * k] = (uint8_t)bv[hf][k];
      }
#pragma unroll
      for (int k = 0; k < 9; ++k)
        if (m + 4 * k <= kSlab) Hs[(m + 4 * k + 1) * kCS + 3] = join(tv[0][k], tv[1][k]);
#pragma unroll
      for (int r = 0; r < kRows; ++r) Gs[r] = join(w[0][r], w[1][r]);
      prev = join(cw[0], cw[1]);
      uint4* col0 = reinterpret_cast<uint4*>(Hs + kCS + 8 * m + 4);
      col0[0] = make_uint4(Gs[0], Gs[1], Gs[2], Gs[3]);
      col0[1] = make_uint4(Gs[4], Gs[5], Gs[6], Gs[7]);
      if (m > 0) Hs[8 * m + 3] = prev;  // corner: row 8m-1, column c = -1
    }
    __syncwarp();
    clk.lap(2);
    {
      const uint32_t bA = bs32 + (3 - m), bB = bs32 + kBS + (3 - m);
#pragma unroll 4
      for (int c = 1; c <= kSlab; ++c) {
        const uint32_t topv = Hs[(c + 1) * kCS + 3];
        const uint32_t fa = __shfl_up_sync(full, Gs[kRows - 1], 1, 4);
        const uint32_t Gu = m == 0 ? topv : fa;
        const uint32_t Gd = prev;
        prev = Gu;
        const uint32_t ca = lds_u8(bA + c), cb = lds_u8(bB + c);
        uint32_t Xv[kRows];
#pragma unroll
        for (int r = 0; r < kRows; ++r) {
          const uint32_t sg = prmt((uint32_t)lds_s8(sa[0][r] + ca), (uint32_t)lds_s8(sa[1][r] + cb), 0x5410u);
          Xv[r] = __viaddmax_s16x2(r == 0 ? Gd : Gs[r - 1], sg, __viaddmax_s16x2(Gs[r], NEG_G2, NEG_G2));
        }
        uint32_t gg = Gu;
#pragma unroll
        for (int r = 0; r < kRows; ++r) {
          gg = __viaddmax_s16x2(gg, NEG_G2, Xv[r]);
          Gs[r] = gg;
        }
        uint4* col = reinterpret_cast<uint4*>(Hs + (c + 1) * kCS + 8 * m + 4);
        col[0] = make_uint4(Gs[0], Gs[1], Gs[2], Gs[3]);
        col[1] = make_uint4(Gs[4], Gs[5], Gs[6], Gs[7]);
      }
    }
    __syncwarp();
    clk.lap(3);
    // 5) searching halves: first row-major cell of the lane band holding the score
#pragma unroll
    for (int hf = 0; hf < 2; ++hf) {
      TbHalf& X = H[hf];
      const bool srch = X.mode == 1 && X.on;
      const int m8 = (X.band & 31) & 3;
      int key = 1 << 30;  // r * 64 + c
      if (srch) {
        const int target = X.best - g;
        for (int c = m + 1; c <= kSlab; c += 4) {
          const uint4* col = reinterpret_cast<const uint4*>(Hs + (c + 1) * kCS + 8 * m8 + 4);
          const uint4 v0 = col[0], v1 = col[1];
          const uint32_t vv[8] = {v0.x, v0.y, v0.z, v0.w, v1.x, v1.y, v1.z, v1.w};
#pragma unroll
          for (int r = kRows - 1; r >= 0; --r) {
            const int i = R0[hf] + 8 * m8 + r + 1, j = D[hf] + c - m8;
            if (half16(vv[r], hf) == target && i <= X.la && j >= 1 && j <= X.lb) key = min(key, r * 64 + c);
          }
        }
      }
      key = min(key, __shfl_xor_sync(full, key, 1));
      key = min(key, __shfl_xor_sync(full, key, 2));
      if (srch) {
        if (key < (1 << 30)) {
          const int r = key >> 6, c = key & 63;
          const long long k2 = ((long long)(R0[hf] + 8 * m8 + r + 1) << 32) | (long long)(D[hf] + c - m8);
          if (X.found < 0 || k2 < X.found) X.found = k2;
        }
        X.scur = X.cand + 1;
        X.cand = -1;
      }
    }
    clk.lap(4);
    // 6) walking halves: lane m == half walks its problem through the block
    if (m < 2) {
      const int hf = m;
      int mode = hf ? H[1].mode : H[0].mode;
      if (mode == 2) {
        int i = hf ? H[1].i : H[0].i, j = hf ? H[1].j : H[0].j, h = hf ? H[1].h : H[0].h, n = hf ? H[1].n : H[0].n;
        const int r0 = hf ? R0[1] : R0[0], d0 = hf ? D[1] : D[0];
        const int64_t p = hf ? H[1].p : H[0].p;
        uint8_t* o = out + (p - first) * stride;
        const uint8_t* as = aS + hf * kBlk - r0 - 1;   // as[i] = a[i - 1] for rows of the block
        const uint8_t* bs = bS + hf * kBS - d0 + 3;    // bs[j] = b[j - 1] for columns D-3 .. D+36
        uint8_t* ops = opsS + hf * kOpsCap;
        const int sh16 = 16 * hf;
        int t = i - r0 - 1;
        int c = j - d0 + (t >> 3);
        while (h > 0 && t >= 0 && c >= 1) {
          const int cu = c - ((t > 0 && (t & 7) == 0) ? 1 : 0);  // row above: one column left at a lane start
          const uint32_t* up_col = Hs + (cu + 1) * kCS + t + 3;     // (t-1, cu)
          const int uV = (int)(int16_t)(up_col[0] >> sh16) + g;
          const int dV = (int)(int16_t)(up_col[-kCS] >> sh16) + g;
          const int lV = (int)(int16_t)(Hs[c * kCS + t + 4] >> sh16) + g;
          const int ra = as[i], rb = bs[j];
          const int sub = sig_s[ra * 32 + rb];
          const bool isD = h == dV + sub;
          const bool isU = !isD && h == uV - g;
          const bool mvI = isD || isU;
          const uint8_t op = isD ? (ra == rb ? 'M' : 'X') : (isU ? 'D' : 'I');
          h = isD ? dV : (isU ? uV : lV);
          i -= mvI ? 1 : 0;
          j -= isU ? 0 : 1;
          c = isD ? cu - 1 : (isU ? cu : c - 1);
          t -= mvI ? 1 : 0;
          if (n < kOpsCap) ops[n] = op;
          else if (n < stride) o[stride - 1 - n] = op;  // long paths: the row's tail, moved at the end
          ++n;
        }
        if (hf) { H[1].i = i; H[1].j = j; H[1].h = h; H[1].n = n; if (h <= 0) H[1].mode = 0; }
        else { H[0].i = i; H[0].j = j; H[0].h = h; H[0].n = n; if (h <= 0) H[0].mode = 0; }
      }
    }
    // the walkers' state to their groups
#pragma unroll
    for (int hf = 0; hf < 2; ++hf) {
      const int src = (lane & ~3) | hf;
      TbHalf& X = H[hf];
      X.i = __shfl_sync(full, X.i, src);
      X.j = __shfl_sync(full, X.j, src);
      X.h = __shfl_sync(full, X.h, src);
      X.n = __shfl_sync(full, X.n, src);
      X.mode = __shfl_sync(full, X.mode, src);
    }
    __syncwarp();
    clk.lap(5);
  }
  // 7) outputs, start -> end: op q (walk order) goes to position n-1-q. Ops q < cap are in
  // shared memory; longer paths left ops q >= cap at the row's tail (position stride-1-q),
  // which is shifted left first (ordered 4-byte chunks: every read precedes the overlapping writes).
  __syncwarp();
#pragma unroll
  for (int hf = 0; hf < 2; ++hf) {
    const TbHalf& X = H[hf];
    const bool mine = X.p >= first && X.p < first + count;
    const int64_t q = X.p - first;
    const bool active = X.best > 0 && X.la > 0 && X.lb > 0;
    const int n = active ? X.n : 0;
    const bool overflow = n > stride;
    uint8_t* o = out + (mine ? q : 0) * stride;
    if (mine && !overflow && n > kOpsCap) {
      const int64_t s0 = stride - n;
      for (int64_t u0 = 0; u0 < n - kOpsCap; u0 += 4) {
        const int64_t u = u0 + m;
        const uint8_t v = u < n - kOpsCap ? o[s0 + u] : 0;
        __syncwarp(0xfu << (lane & ~3));
        if (u < n - kOpsCap) o[u] = v;
        __syncwarp(0xfu << (lane & ~3));
      }
    }
    if (mine && !overflow) {
      const uint8_t* ops = opsS + hf * kOpsCap;
      for (int u = max(0, n - kOpsCap) + m; u < n; u += 4) o[u] = ops[n - 1 - u];
    }
    if (mine && m == 0) {
      out_len[q] = overflow ? -1 : (int32_t)n;
      if (coords) {
        coords[4 * q] = active ? X.i : 0; coords[4 * q + 1] = active ? X.j : 0;
        coords[4 * q + 2] = active ? X.ei : 0; coords[4 * q + 3] = active ? X.ej : 0;
      }
    }
  }
  clk.lap(6);
  clk.flush(lane);
}

size_t tb3_smem_bytes() { return 1024 + 8 * kGS * 4 + 8 * 2 * kBS + 8 * 2 * kBlk + 8 * 2 * kOpsCap; }

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
  *slabbest = 2 * groups * *strips * *nslab * 32 + groups * *strips * 32;  // slab maxima, corners, strip maxima
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
  ++*launches;
  const size_t smem = tb3_smem_bytes();
  cudaError_t e = cudaFuncSetAttribute(k_sw16_tb3, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  e = cudaFuncSetAttribute(k_sw16_tb3, cudaFuncAttributePreferredSharedMemoryCarveout, 100);
  if (e != cudaSuccess) return e;
  const int64_t groups = ((first + count - 1) >> 1) - (first >> 1) + 1;
  k_sw16_tb3<<<(unsigned)((groups + 7) / 8), 32, smem, s>>>(A, first, count, out, stride, out_len, coords);
  return cudaGetLastError();
}

}  // namespace dpk
