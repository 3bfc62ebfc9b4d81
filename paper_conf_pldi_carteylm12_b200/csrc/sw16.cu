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
// every column) and, after every block of kSlab = 16 steps, every lane's 8 rows at the
// column it is on (a staircase, column 16 s - lane: warp-uniform, coalesced,
// no per-step branch), the G above it there and its best G over the block
// (0.25 + 0.5 B/cell), plus every lane's maximum over the strip. k_sw16_tb5 recomputes
// only the 32x32 (sheared) blocks the canonical traceback needs, as 2-bit
// direction codes that carry the oracle's tie-break (stop at H = 0, then
// diag > up > left; end cell = first maximum in row-major order), and walks them.
#include <algorithm>
#include <cstdint>
#include <cstdlib>
#include <cuda_runtime.h>

#include "dp_internal.h"

namespace dpk {
namespace {

#ifndef SW16_UNROLL
#define SW16_UNROLL 16  // steady-loop unroll (2 / 4 / 8 / 16 / 32: sweep 1.344 / 1.268 / 1.234 / 1.225 / 1.224 ms)
#endif
constexpr int kRows = 8;              // rows per lane
constexpr int kStrip = 32 * kRows;    // rows per strip
#ifndef SW16_BAND
#define SW16_BAND 16
#endif
constexpr int kBand = SW16_BAND;      // checkpoint band height (16: two lanes, 8: every lane)
constexpr int kLanesPerBand = kBand / kRows;
constexpr int kBandsPerStrip = kStrip / kBand;
#ifndef SW16_SLAB
#define SW16_SLAB 16
#endif
constexpr int kSlab = SW16_SLAB;      // checkpoint column spacing (sweep steps)
constexpr int kBW = 32;               // traceback block width (re-run steps): two checkpoint intervals
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
    // only lane 0 reads the boundary word (any other lane's read would race with lane 31 rewriting
    // that column's word a few steps later)
    uint32_t bw = NEG_G2;
    if (lane0 && from_bnd && live) bw = lds_u32_v(rec + 4);
    Gu = lane0 ? bw : fa;
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
  // sigma transposed, sigT[c][a] (32 x 32 int8): kDead outside the alphabet, so a = 31 is a
  // dead residue and c = asz a dead column code
  int8_t* sigT = reinterpret_cast<int8_t*>(smem);
  constexpr int sig_bytes = 32 * 32;
  for (int q = threadIdx.x; q < 32 * 32; q += blockDim.x) {
    const int c = q >> 5, a = q & 31;
    sigT[q] = (c < asz && a < asz) ? A.sigma[a * asz + c] : (int8_t)kDead;
  }
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
  const bool lane0 = lane == 0, odd = (lane + 1) % kLanesPerBand == 0;  // "odd": the lane ends a band
  FwdState S;
  S.best2 = NEG_G2;  // max G = max h - g

  for (int st = 0; st < strips; ++st) {
    const int i0 = st * kStrip + lane * kRows;  // 0-based index of my first row
    // profiles for my 8 rows: P[c][row] int8, one 8-byte word per lane per residue. Each 4-row
    // word is gathered from column c of sigT with byte permutes: residue a selects byte a & 7 of
    // the 8-byte window a >> 3, one PRMT per window, merged under per-row window masks.
    uint32_t sel[4], msk[4][4];  // [problem A rows 0-3, 4-7, problem B rows 0-3, 4-7]
#pragma unroll
    for (int g4 = 0; g4 < 4; ++g4) {
      const uint8_t* src = g4 < 2 ? aA : aB;
      const int la = g4 < 2 ? laA : laB;
      uint32_t sl = 0, m[4] = {0, 0, 0, 0};
#pragma unroll
      for (int k = 0; k < 4; ++k) {
        const int i = i0 + 4 * (g4 & 1) + k;
        const int a = i < la ? src[i] : 31;  // dead rows read sigma = kDead
        sl |= (uint32_t)(a & 7) << (4 * k);
        m[a >> 3] |= 0xffu << (8 * k);
      }
      sel[g4] = sl;
#pragma unroll
      for (int w = 0; w < 4; ++w) msk[g4][w] = m[w];
    }
    for (int c = 0; c <= asz; ++c) {
      uint32_t col[8];  // sigT[c][0..31]
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
    // Steps come in blocks of kSlab (one slab); after block s every lane checkpoints
    // at once (warp-uniform, coalesced): its 8 G values at column kSlab (s+1) - lane,
    // the G above it there (corner), and its best G over the block.
    const uint32_t rec0 = sh_rec + kRec * (kPad - lane);
    const int K = lbm + 31;
    constexpr int U = SW16_UNROLL;
    constexpr int kB = TB ? kSlab : 2 * kSlab;  // steps per block (score only: no checkpoints)
    for (int kb = 0, sl = 0; kb < K; kb += kB, ++sl) {
      const int ke = min(kb + kB, K);
      if (kB == U && kb >= 31 && ke <= lbm - 1) {  // a whole steady block: one unrolled run
        const uint32_t rec = rec0 + kRec * kb;
        uint32_t* rk = rowck + (kb - lane);
#pragma unroll
        for (int u = 0; u < U; ++u)
          sw_step<TB, false, MULTI>(S, rec + kRec * u, kb + u - lane + 1, lbm, lane0, odd, spill31, from_bnd, NEG_G2,
                                    laneA, laneB, rk + u);
        if (MULTI) __syncwarp();
      } else {
      // steady range: lane 31 at j >= 1 and lane 0 at j <= lbm - 1
      const int s0 = min(max(kb, 31), ke), s1 = max(s0, min(ke, lbm - 1));
      int k = kb;
      for (; k < s0; ++k) {
        sw_step<TB, true, MULTI>(S, rec0 + kRec * k, k - lane + 1, lbm, lane0, odd, spill31, from_bnd, NEG_G2,
                                 laneA, laneB, rowck + (k - lane));
        // lane 0 reads column j's boundary word at step j - 1, lane 31 rewrites it at step j + 30: a
        // __syncwarp at least every 31 steps orders the two (MULTI: more than one strip of rows)
        if (MULTI) __syncwarp();
      }
      for (; k + U <= s1; k += U) {
        const uint32_t rec = rec0 + kRec * k;
        uint32_t* rk = rowck + (k - lane);
#pragma unroll
        for (int u = 0; u < U; ++u)
          sw_step<TB, false, MULTI>(S, rec + kRec * u, k + u - lane + 1, lbm, lane0, odd, spill31, from_bnd, NEG_G2,
                                    laneA, laneB, rk + u);
        if (MULTI) __syncwarp();
      }
      for (; k < s1; ++k) {
        sw_step<TB, false, MULTI>(S, rec0 + kRec * k, k - lane + 1, lbm, lane0, odd, spill31, from_bnd, NEG_G2,
                                  laneA, laneB, rowck + (k - lane));
        if (MULTI) __syncwarp();
      }
      for (; k < ke; ++k) {
        sw_step<TB, true, MULTI>(S, rec0 + kRec * k, k - lane + 1, lbm, lane0, odd, spill31, from_bnd, NEG_G2,
                                 laneA, laneB, rowck + (k - lane));
        if (MULTI) __syncwarp();
      }
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
// k_sw16_tb5: persistent warps of 8 four-lane groups; CTAs of kTbWarps warps
// share the sigma table. Each group carries two problems, one per s16x2 half:
// the low half serves even problems, the high half odd ones (the forward packed
// problems 2g, 2g+1 into the halves of its checkpoints), and each half takes its
// next problem from its own queue (an atomic counter) as soon as it is done, so
// warps stay full until the queues drain.
//
// A traceback "block" is 32 rows (forward lanes L0..L0+3 of one strip,
// L0 = 4 (blk mod 8)) x two slabs from checkpoint sl (kBW = 32 steps): forward lane L0+m covered
// columns j = D + c - m, c = 1..32, D = 16 sl - L0, at forward steps 16 sl + c - 1 (a walker's
// block starts at the checkpoint that leaves it 17..32 columns of room).
// So in the sheared column c all four lanes are at the SAME forward step and
// group lane m re-runs forward lane L0+m (8 rows) for 32 steps exactly as the
// sweep did (no ramp): the left column is its checkpoint, its first diagonal the
// corner word, lane 0's "up" the band checkpoint row above the block.
//
// The re-run computes KEYS K = 4 G + code instead of G: every candidate of the
// cell carries its traceback priority in the two low bits (Z: H = 0 -> 3,
// diagonal 2, up 1, left 0; sigma is tabulated as 4 sigma + 2), so the max that
// the recurrence takes anyway also takes the oracle's tie-break (stop at H = 0,
// then diag > up > left). Only the codes are kept: 2 bits per cell and problem,
// one 32-bit word per lane and column (8 rows x 2 halves), 512 B per group, and
// the walk reads one word per step. Keys stay in s16 while 4 x the score bound
// fits (plan check). The end cell (first row-major maximum) comes from the
// per-lane strip maxima, then the slabs of that lane whose maximum equals the
// score, then a compare inside the re-run (taken only on a hit).
constexpr int kTbWarps = 4;              // warps per CTA
#ifndef TB_GL
#define TB_GL 4                          // lanes per group = forward lanes per traceback block (2 measured slower)
#endif
constexpr int kGL = TB_GL;               // 2: blocks of 16 rows (one checkpoint band), 4: 32 rows
constexpr int kGroups = 32 / kGL;        // groups per warp
constexpr int kBlk = kRows * kGL;        // traceback block height
#ifndef TB5_UNROLL
#define TB5_UNROLL 1   // 1 / 2 / 4 / 8 / 32: traceback 1.06 / 1.10 / 1.16 / 1.22 / 1.63 ms (register pressure)
#endif
constexpr int kTbUnroll = TB5_UNROLL;   // re-run steps unrolled
#ifndef TB5_MINB
#define TB5_MINB 4                       // CTAs per SM (register cap; 4 / 5 / 6 with no unroll: 1.049 / 1.059 / 1.099 ms)
#endif
constexpr int kSigRow = 34;              // int16 per sigma row (17 words: see k_sw16_tb5)
constexpr int kSigBytes = ((32 * kSigRow * 2 + 127) / 128) * 128;
constexpr int kCW = kGL * kBW;           // code words per group: [c - 1][m]
constexpr int kCWp = kCW + 4;            // group stride: 4 banks apart, so the 8 groups' code stores hit 32 banks
constexpr int kTS = 36;                  // top-row keys per group, c = 0..32
constexpr int kBS = 40;                  // staged b residues per half (columns D-3 .. D+36)
constexpr int kDeadCode = 31;            // residue code whose sigma row/column is kDead4 (alphabets < 32)
constexpr int kDead4 = -4000;            // keyed sigma outside a problem
constexpr uint32_t kClean = 0xfffcfffcu, kCodeBits = 0x00030003u;

enum : int { kIdle = 0, kSearch = 1, kWalk = 2, kFinish = 3, kDone = 4 };
struct TbState {      // one problem in one half of a group (shared memory; written by one lane)
  long long p;        // problem id
  long long found;    // search: row-major key (i << 32 | j) of the first maximum, -1 none
  const uint8_t *a, *b;  // residues
  int la, lb, best;
  int mode;
  int band;           // search: first lane band (strip * 32 + lane) whose maximum is the score
  int scur, cand;     // search: next slab to probe, candidate slab (-1 none)
  unsigned cbits;     // search: candidate slabs scur + b of the current probe window still to visit
  int i, j, n;        // walk: current cell, ops written
  int ei, ej;         // end cell
};
constexpr int kGroupBytes = 4 * kCWp + 4 * kTS + 2 * kBS + 2 * kBlk + 2 * (int)sizeof(TbState);
constexpr int kTbWarpBytes = kGroups * kGroupBytes;

// first forward lane of the search block of lane band ln (ln in the block's lane 2 or 3 when ln >= 2)
__device__ __forceinline__ int search_l0(int ln) { return ln < 2 ? 0 : ((ln - 2) & ~1); }
__device__ __forceinline__ uint32_t lds_u8(uint32_t a) {
  uint32_t v;
  asm("ld.shared.u8 %0, [%1];" : "=r"(v) : "r"(a));
  return v;
}
__device__ __forceinline__ uint32_t lds_s16w(uint32_t a) {
  int v;
  asm("ld.shared.s16 %0, [%1];" : "=r"(v) : "r"(a));
  return (uint32_t)v;
}
__device__ __forceinline__ uint32_t lds_u32(uint32_t a) {
  uint32_t v;
  asm volatile("ld.shared.u32 %0, [%1];" : "=r"(v) : "r"(a) : "memory");
  return v;
}
__device__ __forceinline__ void sts_u32(uint32_t a, uint32_t v) {
  asm volatile("st.shared.u32 [%0], %1;" ::"r"(a), "r"(v) : "memory");
}
__device__ __forceinline__ uint32_t join(uint32_t lo_src, uint32_t hi_src) { return prmt(lo_src, hi_src, 0x7610u); }
__device__ __forceinline__ uint32_t key4(uint32_t g2) { return (g2 << 2) & kClean; }  // 4 G per half
__device__ __forceinline__ uint32_t pack2(int v) { return (uint32_t)(uint16_t)(int16_t)v * 0x10001u; }
__device__ __forceinline__ void prefetch_l2(const void* p) { asm volatile("prefetch.global.L2 [%0];" ::"l"(p)); }

__global__ void __launch_bounds__(kTbWarps * 32, TB5_MINB) k_sw16_tb5(Sw16Args A, int64_t first, int64_t count,
                                                                       uint8_t* out, int64_t stride, int32_t* out_len,
                                                                       int32_t* coords) {
  extern __shared__ __align__(16) uint8_t tsm[];
  // [32][kSigRow] 4 sigma + 2, kDead4 outside the alphabet. Rows 17 words apart: a lookup's bank
  // is (17 a + b / 2) mod 32, so the rows of a group's lanes (same b, different a) spread over
  // the banks (with 16-word rows a only chose between two banks)
  int16_t* sig_s = reinterpret_cast<int16_t*>(tsm);
  for (int q = threadIdx.x; q < 32 * kSigRow; q += blockDim.x) {
    const int x = q / kSigRow, y = q % kSigRow;
    sig_s[q] = (x < A.asz && y < A.asz) ? (int16_t)(4 * A.sigma[x * A.asz + y] + 2) : (int16_t)kDead4;
  }
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31, gq = lane / kGL, m = lane % kGL;
  uint8_t* wb = tsm + kSigBytes + warp * kTbWarpBytes;
  uint32_t* Cs = reinterpret_cast<uint32_t*>(wb) + gq * kCWp;
  uint32_t* Ts = reinterpret_cast<uint32_t*>(wb + kGroups * 4 * kCWp) + gq * kTS;
  uint8_t* bS = wb + kGroups * 4 * (kCWp + kTS) + gq * 2 * kBS;                  // [2][kBS] staged b residues
  uint8_t* aS = wb + kGroups * (4 * (kCWp + kTS) + 2 * kBS) + gq * 2 * kBlk;  // [2][kBlk] staged a residues
  TbState* St = reinterpret_cast<TbState*>(wb + kGroups * (4 * (kCWp + kTS) + 2 * kBS + 2 * kBlk)) + 2 * gq;
  const uint32_t sig32 = (uint32_t)__cvta_generic_to_shared(sig_s);
  const uint32_t cs32 = (uint32_t)__cvta_generic_to_shared(Cs);
  const uint32_t ts32 = (uint32_t)__cvta_generic_to_shared(Ts);
  const uint32_t bs32 = (uint32_t)__cvta_generic_to_shared(bS);
  const uint32_t aS32 = (uint32_t)__cvta_generic_to_shared(aS);
  const unsigned full = 0xffffffffu, gmask = ((1u << kGL) - 1) << (lane & ~(kGL - 1));
  const int g = A.gap;
  const uint32_t NEG_G2 = pack2(-g), NEG4 = pack2(-4 * g), NEG4U = pack2(-4 * g + 1), ZC = pack2(-4 * g + 3);
  const int64_t SM = A.strips_max, NS = A.nslab_max;
  // queues: half hf serves problems p = 2 k + hf in [first, first + count)
  const int64_t k0[2] = {(first + 1) >> 1, first >> 1};
  const int64_t kn[2] = {((first + count + 1) >> 1) - k0[0], ((first + count) >> 1) - k0[1]};
  if (m == 0) { St[0].mode = kIdle; St[1].mode = kIdle; }
  __syncthreads();
  PhaseClock clk;
  clk.dbg = A.dbg;
  clk.start();

  for (;;) {
    // A) idle halves take their next problem; a problem with score 0 finishes at once
#pragma unroll
    for (int hf = 0; hf < 2; ++hf) {
      const bool idle = St[hf].mode == kIdle;
      __syncwarp(gmask);  // every lane of the group has read the mode before lane 0 rewrites the state
      if (!idle) continue;
      int64_t q = 0;
      if (m == 0) q = atomicAdd(reinterpret_cast<unsigned long long*>(A.tb_ctr) + hf, 1ull);
      q = __shfl_sync(gmask, q, lane & ~(kGL - 1));
      if (m == 0) {
        TbState& S = St[hf];
        if (q >= kn[hf]) {
          S.mode = kDone;
        } else {
          const int64_t p = 2 * (k0[hf] + q) + hf;
          S.p = p;
          const int64_t ao = A.a_off[p], bo = A.b_off[p];
          S.a = A.a_cat + ao;
          S.b = A.b_cat + bo;
          S.la = (int)(A.a_off[p + 1] - ao);
          S.lb = (int)(A.b_off[p + 1] - bo);
          S.best = A.scores[p];
          S.mode = (S.best > 0 && S.la > 0 && S.lb > 0) ? kSearch : kFinish;
          S.band = -1; S.scur = 0; S.cand = -1; S.found = -1;
          S.i = S.j = S.n = S.ei = S.ej = 0;
        }
      }
      __syncwarp(gmask);
      // prologue: first lane band (row-major: strip, lane) whose strip maximum reaches the score
      if (St[hf].mode == kSearch) {
        const int64_t grp = St[hf].p >> 1;
        const int best = St[hf].best, la = St[hf].la;
        int band = -1;
        for (int st = 0; st * kStrip < la && band < 0; ++st) {
          int firstl = 32;
#pragma unroll
          for (int q8 = 32 / kGL - 1; q8 >= 0; --q8)
            if (half16(__ldcg(A.lanebest + (grp * SM + st) * 32 + (32 / kGL) * m + q8), hf) + g == best)
              firstl = (32 / kGL) * m + q8;
#pragma unroll
          for (int o = 1; o < kGL; o <<= 1) firstl = min(firstl, __shfl_xor_sync(gmask, firstl, o));
          if (firstl < 32) band = st * 32 + firstl;
        }
        __syncwarp(gmask);
        if (m == 0) {
          St[hf].band = band;
          if (band < 0) St[hf].mode = kFinish;  // cannot happen: the maxima name the score
        }
        __syncwarp(gmask);
      }
    }
    if (!__any_sync(full, St[0].mode != kDone || St[1].mode != kDone)) break;
    clk.lap(0);
    // B) searching halves: next candidate slab of their lane band (32 slabs per probe)
#pragma unroll
    for (int hf = 0; hf < 2; ++hf) {
      while (St[hf].mode == kSearch && St[hf].cand < 0) {
        const TbState& S = St[hf];
        const int64_t grp = S.p >> 1;
        const int nsl = (S.lb + 31 + kSlab - 1) / kSlab, scur = S.scur, best = S.best;
        const uint32_t* sb = A.slabbest + ((grp * SM + (S.band >> 5)) * NS) * 32 + (S.band & 31);
        uint32_t bits = 0;
#pragma unroll
        for (int q = 0; q < 32 / kGL; ++q) {
          const int s = scur + m + kGL * q;
          if (s < nsl && half16(__ldcg(sb + (int64_t)s * 32), hf) + g == best) bits |= 1u << (m + kGL * q);
        }
#pragma unroll
        for (int o = 1; o < kGL; o <<= 1) bits |= __shfl_xor_sync(gmask, bits, o);
        __syncwarp(gmask);
        if (m == 0) {
          TbState& W = St[hf];
          if (bits) {
            W.cand = scur + __ffs(bits) - 1;
            W.cbits = bits;
          } else {
            W.scur = scur + 32;
            if (W.scur >= nsl) {  // candidates exhausted: walk from the first maximum
              if (W.found >= 0) {
                W.mode = kWalk;
                W.i = W.ei = (int)(W.found >> 32);
                W.j = W.ej = (int)(W.found & 0xffffffffll);
              } else {
                W.mode = kFinish;  // cannot happen
              }
            }
          }
        }
        __syncwarp(gmask);
      }
    }
    __syncwarp();
    clk.lap(1);
    clk.count(7);
    // C) this round's block per half, D) prefetch, E) checkpoints as keys. Every global
    // load of the round is issued before any shared-memory store.
    int R0[2], D[2];
    uint32_t sa[2][kRows];
    uint32_t Kc[kRows], prev;
    uint32_t T4m1 = 0x7fff7fffu;  // search target 4 (best - g) - 1 in lane m8's half, else never exceeded
    {
      uint32_t w[2][kRows], cw[2];
#pragma unroll
      for (int hf = 0; hf < 2; ++hf) {
        const TbState& S = St[hf];
        const int mode = S.mode;
        const bool srch = mode == kSearch && S.cand >= 0;
        const bool on = srch || mode == kWalk;
        const int64_t grp = S.p >> 1;
        // block rows R0+1 .. R0+32 = forward lanes L0..L0+3 of one strip, L0 even (the top row is
        // a band checkpoint). A walker's block puts it in lane L0+2 or L0+3, so it runs through
        // at least 16 rows before leaving upwards.
        int r0 = 0, sl = 0;
        if (srch) {
          // the search block puts the band in its lane 2 or 3 and the candidate slab in its second
          // half, so a walk starting in this round from the end cell has room above and to the left
          const int lnb = S.band & 31, L0b = search_l0(lnb);
          r0 = (S.band >> 5) * kStrip + kRows * L0b;
          sl = max(0, S.cand - (kBW / kSlab - 1));
          if (m == lnb - L0b) {
            const uint32_t t = (uint32_t)(uint16_t)(int16_t)(4 * (S.best - g) - 1);
            T4m1 = hf ? ((T4m1 & 0xffffu) | (t << 16)) : ((T4m1 & 0xffff0000u) | t);
          }
        } else if (mode == kWalk) {
          const int ln = ((S.i - 1) % kStrip) / kRows;
          r0 = (S.i - 1) / kStrip * kStrip +
               kRows * (kBand == kRows ? (ln < kGL - 1 ? 0 : ln - (kGL - 1))  // walker in the block's last lane
                                       : (kGL == 2 ? (ln & ~1) : (ln < 2 ? 0 : ((ln - 2) & ~1))));
          // the block starts at a checkpoint (every kSlab steps) that puts the walker at c in
          // [kBW - kSlab + 1, kBW]: at least kSlab columns of room before leaving on the left
          sl = max(0, (S.j + ln - 1) / kSlab - (kBW / kSlab - 1));
          // the next block is left (same rows or 16 up) or 32 rows up: pull their checkpoints into L2
#pragma unroll
          for (int q = 0; q < 3; ++q) {
            const int nr = r0 - (q == 0 ? 0 : (q == 1 ? 16 : 32)), ns = sl - (q == 0 ? kBW / kSlab : (q == 1 ? 1 : 0));
            if (nr < 0 || ns < 1) continue;
            const int st = nr / kStrip, L0 = (nr % kStrip) / kRows;
            const int64_t base = (grp * SM + st) * NS + (ns - 1);
            prefetch_l2(A.colck + base * kStrip + (L0 + m) * kRows);
            if (m == 0) prefetch_l2(A.corner + base * 32 + L0);
            if (nr > 0) {
              const int bnd = nr / kBand - 1, j0 = max(1, ns * kSlab - L0 + (32 / kGL) * m);
              if (j0 <= S.lb)
                prefetch_l2(A.rowck + ((grp * SM + bnd / kBandsPerStrip) * kBandsPerStrip + bnd % kBandsPerStrip) *
                                          A.max_lb + (j0 - 1));
            }
          }
        }
        R0[hf] = r0;
        const int st = r0 / kStrip, L0 = (r0 % kStrip) / kRows, l = L0 + m;
        D[hf] = sl * kSlab - L0;
        const bool ck = on && sl > 0;
        const int64_t base = (grp * SM + st) * NS + (ck ? sl - 1 : 0);
        const uint4* cp = reinterpret_cast<const uint4*>(A.colck + base * kStrip + l * kRows);
        const uint4 v0 = ck ? __ldcg(cp) : make_uint4(NEG_G2, NEG_G2, NEG_G2, NEG_G2);
        const uint4 v1 = ck ? __ldcg(cp + 1) : make_uint4(NEG_G2, NEG_G2, NEG_G2, NEG_G2);
        w[hf][0] = v0.x; w[hf][1] = v0.y; w[hf][2] = v0.z; w[hf][3] = v0.w;
        w[hf][4] = v1.x; w[hf][5] = v1.y; w[hf][6] = v1.z; w[hf][7] = v1.w;
        cw[hf] = ck ? __ldcg(A.corner + base * 32 + l) : NEG_G2;
        const uint8_t* ap = S.a;
        const uint8_t* bp = S.b;
        const int la = S.la, lb = S.lb;
        uint32_t av[kRows], bv[kBS / kGL], tv[(kBW + kGL) / kGL];
#pragma unroll
        for (int r = 0; r < kRows; ++r) {
          const int i = R0[hf] + kRows * m + r + 1;
          av[r] = (on && i <= la) ? __ldg(ap + i - 1) : (uint32_t)kDeadCode;
        }
#pragma unroll
        for (int k = 0; k < kBS / kGL; ++k) {  // b residues of columns D-3 .. D+36 (x = j - D + 3)
          const int j = D[hf] + m + kGL * k - 3;
          bv[k] = (on && j >= 1 && j <= lb) ? __ldg(bp + j - 1) : (uint32_t)kDeadCode;
        }
        // top row (G of row R0, columns D + c, c = 0..32): the band checkpoint above the block
        const int bnd = R0[hf] / kBand - 1;
        const uint32_t* rk = A.rowck + ((grp * SM + (bnd >= 0 ? bnd / kBandsPerStrip : 0)) * kBandsPerStrip +
                                        (bnd >= 0 ? bnd % kBandsPerStrip : 0)) * A.max_lb - 1;
#pragma unroll
        for (int k = 0; k < (kBW + kGL) / kGL; ++k) {
          const int c = m + kGL * k, j = D[hf] + c;
          tv[k] = (on && bnd >= 0 && c <= kBW && j >= 1 && j <= lb) ? __ldcg(rk + j) : NEG_G2;
        }
        // this half's residues and top-row keys to shared memory
#pragma unroll
        for (int r = 0; r < kRows; ++r) {
          sa[hf][r] = sig32 + 2 * kSigRow * av[r];
          aS[hf * kBlk + kRows * m + r] = (uint8_t)av[r];
        }
#pragma unroll
        for (int k = 0; k < kBS / kGL; ++k) bS[hf * kBS + m + kGL * k] = (uint8_t)bv[k];
        int16_t* ts16 = reinterpret_cast<int16_t*>(Ts) + hf;
#pragma unroll
        for (int k = 0; k < (kBW + kGL) / kGL; ++k)
          if (m + kGL * k <= kBW) ts16[2 * (m + kGL * k)] = (int16_t)(4 * half16(tv[k], hf));
      }
#pragma unroll
      for (int r = 0; r < kRows; ++r) Kc[r] = key4(join(w[0][r], w[1][r]));
      prev = key4(join(cw[0], cw[1]));
    }
    const bool anys = __any_sync(full, T4m1 != 0x7fff7fffu);
    __syncwarp();
    clk.lap(2);
    // F) re-run the 32 forward steps of both blocks in keys; codes to shared memory
    int hkey[2] = {1 << 30, 1 << 30};  // search: first hit r * 64 + c per half
    {
      const uint32_t bA = bs32 + (3 - m), bB = bs32 + kBS + (3 - m);
      const uint32_t cw0 = cs32 + 4 * m;
#pragma unroll kTbUnroll
      for (int c = 1; c <= kBW; ++c) {
        const uint32_t topv = lds_u32(ts32 + 4 * c);
        const uint32_t fa = __shfl_up_sync(full, Kc[kRows - 1], 1, kGL);
        const uint32_t Ku = m == 0 ? topv : fa;
        const uint32_t Kd = prev;
        prev = Ku;
        const uint32_t ca = 2 * lds_u8(bA + c), cb = 2 * lds_u8(bB + c);
        uint32_t Xv[kRows];
#pragma unroll
        for (int r = 0; r < kRows; ++r) {
          const uint32_t sg = prmt(lds_s16w(sa[0][r] + ca), lds_s16w(sa[1][r] + cb), 0x5410u);
          Xv[r] = __viaddmax_s16x2(r == 0 ? Kd : Kc[r - 1], sg, __viaddmax_s16x2(Kc[r], NEG4, ZC));
        }
        uint32_t kk = Ku, code = 0;
#pragma unroll
        for (int r = 0; r < kRows; ++r) {
          const uint32_t K = __viaddmax_s16x2(kk, NEG4U, Xv[r]);
          kk = K & kClean;
          Kc[r] = kk;
          code = code * 4u + (K & kCodeBits);
        }
        sts_u32(cw0 + 4 * kGL * (c - 1), code);
        if (anys) {
          uint32_t mx = __vimax3_s16x2(Kc[0], Kc[1], Kc[2]);
          mx = __vimax3_s16x2(mx, Kc[3], Kc[4]);
          mx = __vimax3_s16x2(mx, Kc[5], Kc[6]);
          mx = __vmaxs2(mx, Kc[7]);
          if (__vmaxs2(mx, T4m1) != T4m1) {  // rare: a cell of this lane reaches the score
#pragma unroll
            for (int hf = 0; hf < 2; ++hf) {
              const int th = half16(T4m1, hf), la = St[hf].la, lb = St[hf].lb;
#pragma unroll
              for (int r = 0; r < kRows; ++r) {
                const int i = R0[hf] + kRows * m + r + 1, j = D[hf] + c - m;
                if (half16(Kc[r], hf) > th && i <= la && j >= 1 && j <= lb) hkey[hf] = min(hkey[hf], r * 64 + c);
              }
            }
          }
        }
      }
    }
    __syncwarp();
    clk.lap(3);
    // G) searching halves: first row-major cell of the lane band holding the score
#pragma unroll
    for (int hf = 0; hf < 2; ++hf) {
      int key = hkey[hf];
#pragma unroll
      for (int o = 1; o < kGL; o <<= 1) key = min(key, __shfl_xor_sync(full, key, o));
      TbState& S = St[hf];
      if (m == 0 && S.mode == kSearch && S.cand >= 0) {
        if (key < (1 << 30)) {
          const int m8 = (S.band & 31) - search_l0(S.band & 31), r = key >> 6, c = key & 63;
          const long long k2 = ((long long)(R0[hf] + kRows * m8 + r + 1) << 32) | (long long)(D[hf] + c - m8);
          if (S.found < 0 || k2 < S.found) S.found = k2;
        }
        const unsigned rest = S.cbits & ~(1u << (S.cand - S.scur));
        const int nsl = (S.lb + 31 + kSlab - 1) / kSlab;
        if (rest) {              // the next candidate of this probe window
          S.cbits = rest;
          S.cand = S.scur + __ffs(rest) - 1;
        } else if (S.scur + 32 < nsl) {  // probe the next window
          S.scur += 32;
          S.cand = -1;
        } else {                 // search complete: walk from the first maximum (this round if it is in
          S.mode = kWalk;        // this block: its codes are in shared memory; phase H checks)
          S.i = S.ei = (int)(S.found >> 32);
          S.j = S.ej = (int)(S.found & 0xffffffffll);
        }
      }
    }
    __syncwarp();  // phase G's state updates (lane 0 of a group) before the walkers (lanes 0, 1) read them
    clk.lap(4);
    // H) walking halves: lane m == half walks its problem through the block's codes
    if (m < 2) {
      const int hf = m;
      TbState& S = St[hf];
      if (S.mode == kWalk) {
        int i = S.i, j = S.j;
        const int r0 = R0[hf], d0 = D[hf];
        uint8_t* const o0 = out + (S.p - first) * stride;
        uint8_t* o = o0 + S.n;                            // ops end -> start (stride >= la + lb: no overflow)
        const uint32_t as32 = aS32 + hf * kBlk - r0 - 1;  // a[i - 1] of the block's rows at as32 + i
        const uint32_t bsx = bs32 + hf * kBS - d0 + 3;    // b[j - 1] of columns D-3 .. D+36 at bsx + j
        const uint32_t cw = cs32 - 4 * kGL;               // code word (c, lane mm) at cw + 4 kGL c + 4 mm
        const int sh = 16 * hf + 14;
        int t = i - r0 - 1;
        int c = j - d0 + (t >> 3);
        bool stop = false;
        if (t >= kBlk || c > kBW) t = -1;  // a search just ended outside this block: walk next round
        while (t >= 0 && c >= 1) {
          const uint32_t wd = lds_u32(cw + 4 * kGL * c + 4 * (t >> 3));
          const uint32_t ra = lds_u8(as32 + i), rb = lds_u8(bsx + j);
          const int code = (int)(wd >> (sh - 2 * (t & 7))) & 3;
          if (code == 3) { stop = true; break; }      // H = 0: the alignment starts here
          const bool isD = code == 2, isU = code == 1;
          *o++ = isD ? (ra == rb ? 'M' : 'X') : (isU ? 'D' : 'I');
          const int cu = c - ((t & 7) == 0 && t > 0 ? 1 : 0);  // row above: one column left at a lane start
          const bool mvI = isD || isU;
          i -= mvI ? 1 : 0;
          j -= isU ? 0 : 1;
          c = isD ? cu - 1 : (isU ? cu : c - 1);
          t -= mvI ? 1 : 0;
          if (i == 0 || j == 0) { stop = true; break; }  // table boundary: H = 0
        }
        S.i = i; S.j = j; S.n = (int)(o - o0);
        if (stop) S.mode = kFinish;
      }
    }
    __syncwarp();
    clk.lap(5);
    // I) finished halves: lengths and coordinates (k_sw16_rev reverses the ops afterwards)
#pragma unroll
    for (int hf = 0; hf < 2; ++hf) {
      TbState& S = St[hf];
      if (m == 0 && S.mode == kFinish) {
        const int64_t q = S.p - first;
        out_len[q] = S.n;
        if (coords) {
          coords[4 * q] = S.i; coords[4 * q + 1] = S.j;
          coords[4 * q + 2] = S.ei; coords[4 * q + 3] = S.ej;
        }
        S.mode = kIdle;
      }
    }
    __syncwarp();
    clk.lap(6);
  }
}

// The walk writes each alignment end -> start; one warp per row puts it in order.
__global__ void __launch_bounds__(256) k_sw16_rev(int64_t count, uint8_t* out, int64_t stride, const int32_t* out_len) {
  const int64_t q = (int64_t)blockIdx.x * 8 + (threadIdx.x >> 5);
  const int lane = threadIdx.x & 31;
  if (q >= count) return;
  const int n = out_len[q];
  uint8_t* o = out + q * stride;
  for (int u0 = 0; u0 < n / 2; u0 += 32) {
    const int u = u0 + lane;
    uint8_t x = 0, y = 0;
    if (u < n / 2) { x = o[u]; y = o[n - 1 - u]; }
    __syncwarp();
    if (u < n / 2) { o[u] = y; o[n - 1 - u] = x; }
  }
}

size_t tb5_smem_bytes() { return kSigBytes + (size_t)kTbWarps * kTbWarpBytes; }

}  // namespace

bool sw16_eligible(int64_t max_la, int64_t max_lb, const int8_t* sigma_host, int asz, int gap, bool want_tb) {
  int smax = 0, smin = 0;
  for (int q = 0; q < asz * asz; ++q) { smax = max(smax, (int)sigma_host[q]); smin = min(smin, (int)sigma_host[q]); }
  const int64_t bound = (int64_t)smax * (max_la < max_lb ? max_la : max_lb) + gap;
  // the traceback re-run works on keys 4 G + code (s16): 4 x the bound must fit too
  return asz < 32 && bound < (want_tb ? 7900 : 32000) && smax <= 127 && smin >= -99 && gap >= 1 && gap < 1000 && (asz + 1) * kStrip <= 65535;
}

int sw16_smem_per_warp(int asz, int64_t max_la, int64_t max_lb) {
  const int prof_bytes = (asz + 1) * kStrip;
  const int64_t rec = (max_lb + 2 * kPad) * (max_la > kStrip ? rec_bytes<true>() : rec_bytes<false>());
  return (int)((2 * prof_bytes + rec + 15) & ~15);
}

size_t sw16_smem_bytes(int asz, int64_t max_la, int64_t max_lb) {
  return 32 * 32 + (size_t)kWarps * (size_t)sw16_smem_per_warp(asz, max_la, max_lb);
}

void sw16_state_words(int64_t n, int64_t max_la, int64_t max_lb, int64_t* strips, int64_t* nslab, int64_t* rowck,
                      int64_t* colck, int64_t* slabbest) {
  *strips = (max_la + kStrip - 1) / kStrip;
  *nslab = (max_lb + 31 + kSlab - 1) / kSlab;  // sweep steps lbm + 31 in blocks of kSlab
  const int64_t groups = (n + 1) / 2;
  *rowck = groups * *strips * kBandsPerStrip * max_lb;
  *colck = groups * *strips * *nslab * kStrip;
  *slabbest = 2 * groups * *strips * *nslab * 32 + groups * *strips * 32;  // slab maxima, corners, strip maxima
}

cudaError_t sw16_solve(const Sw16Args& A, bool tb, cudaStream_t s, int64_t* launches) {
  if (A.n == 0) return cudaSuccess;
  const size_t smem = 32 * 32 + (size_t)kWarps * A.smem_per_warp;
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
  const size_t smem = tb5_smem_bytes();
  cudaError_t e = cudaFuncSetAttribute(k_sw16_tb5, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  e = cudaFuncSetAttribute(k_sw16_tb5, cudaFuncAttributePreferredSharedMemoryCarveout, 100);
  if (e != cudaSuccess) return e;
  // persistent grid: as many CTAs as fit, fewer if the queues are short
  static int per_sm = 0, sms = 0;
  if (per_sm == 0) {
    int dev = 0;
    if ((e = cudaGetDevice(&dev)) != cudaSuccess) return e;
    if ((e = cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev)) != cudaSuccess) return e;
    if ((e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k_sw16_tb5, kTbWarps * 32, smem)) != cudaSuccess)
      return e;
    if (per_sm < 1) per_sm = 1;
  }
  const int64_t per_queue = (count + 1) / 2, per_cta = kGroups * kTbWarps;
  const int64_t ctas = std::min<int64_t>((per_queue + per_cta - 1) / per_cta, (int64_t)per_sm * sms);
  if ((e = cudaMemsetAsync(A.tb_ctr, 0, 2 * sizeof(unsigned long long), s)) != cudaSuccess) return e;
  ++*launches;
  k_sw16_tb5<<<(unsigned)ctas, kTbWarps * 32, smem, s>>>(A, first, count, out, stride, out_len, coords);
  if ((e = cudaGetLastError()) != cudaSuccess) return e;
  ++*launches;
  k_sw16_rev<<<(unsigned)((count + 7) / 8), 256, 0, s>>>(count, out, stride, out_len);
  return cudaGetLastError();
}

}  // namespace dpk
