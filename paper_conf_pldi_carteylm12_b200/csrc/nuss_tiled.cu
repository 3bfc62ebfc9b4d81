// Tiled Nussinov (SURVEY.md §8(a) A6b'): the schedule vector (-1,1) of the
// cell-level analysis applied to 32x32 TILES. Tile (I,J) reads tiles (I,K) and
// (K,J) for I < K < J, which are all strictly earlier tile-partitions, so a
// tile-diagonal D = J - I is one hyperplane of independent tiles:
//
//   phase A  C(I,J) = max_{I<K<J} U(I,K) (x) L(K,J)     max-plus tile product,
//            U(I,K)[r][k] = gamma(32I+r, 32K+k), L(K,J)[k][c] = gamma(32K+k+1, 32J+c)
//   phase B  in-tile wavefront over the 63 local anti-diagonals: neighbours,
//            the pair term and the split points k inside tiles I and J.
//
// Phase A is the bulk of the work (n^3/6 split evaluations) and runs as an
// s16x2 max-plus micro-kernel: a warp owns a 32x32 C tile, lane (ty, tx)
// holds rows 4ty..4ty+3 x column pairs 8tx..8tx+7 (16 packed accumulators);
// per k it reads one 16-byte A word (4 rows, each value duplicated into both
// halves) and one 16-byte B word (8 columns) from shared memory and issues 16
// VIADDMNMX.S16x2 (32 split evaluations).
//
// Tables live in global memory (L2-resident), one 4 KB record per tile:
// UT[c][r] = gamma(32I+r, 32J+c) (column-major int16; A operand and in-tile
// reads) and L[k][c] (row-major int16; B operand).
//
// Two drivers share the tile routines:
//   k_nuss_batch  one warp per problem (batches), problems from a length-sorted work queue;
//   k_nuss_grid2  one large problem on the whole grid (cooperative launch): phase A split-K
//                 over the grid's warps with atomicMax into global C, one grid.sync per
//                 tile-diagonal.
// The canonical traceback (Durbin order, smallest k) runs right after the fill
// with the split search spread over a warp.
#include <algorithm>
#include <cstdint>
#include <type_traits>
#include <cooperative_groups.h>
#include <cstdlib>
#include <cuda_runtime.h>

#include "dp_internal.h"

namespace cg = cooperative_groups;

namespace dpk {
namespace {

constexpr int T = 32;
#ifndef NUSS_MICRO_UNROLL
#define NUSS_MICRO_UNROLL 8
#endif
constexpr int kMicroUnroll = NUSS_MICRO_UNROLL;  // phase-A micro-kernel k loop
#ifndef NUSS_WAVE_UNROLL
#define NUSS_WAVE_UNROLL 1   // 1 / 2 / 4: config 5 subset 195 / 233 / 288 ms (registers)
#endif
constexpr int kWaveUnroll = NUSS_WAVE_UNROLL;    // in-tile wavefront steps
#ifndef NUSS_TBW_G
#define NUSS_TBW_G 8   // traceback gamma window (W x W per round trip) and split-search width (32 KC) of the grid
#define NUSS_TBK_G 1   // sweep (16 / 2 measured no faster)
#endif
#ifndef NUSS_TBW_B
#define NUSS_TBW_B 8   // the same for the batch kernel
#define NUSS_TBK_B 1
#endif
constexpr int kTileWords = T * T;      // int16 per tile record half
#ifndef NUSS_GRID_WARPS
#define NUSS_GRID_WARPS 8   // 8 measured best for config 4 (16: 10.6 ms, 12: 9.7, 8: 8.75, 4: 9.3)
#endif
constexpr int kGridWarps = NUSS_GRID_WARPS;  // grid driver
constexpr int kGridMin = 1024;         // single problems longer than this use the whole grid

__host__ __device__ __forceinline__ int64_t tile_id(int I, int J, int nt) {
  return (int64_t)I * nt - (int64_t)I * (I - 1) / 2 + (J - I);
}
__host__ __device__ __forceinline__ int64_t tiles_of(int nt) { return (int64_t)nt * (nt + 1) / 2; }

__device__ __forceinline__ uint32_t dup16(uint32_t w, int hi) {
  uint32_t r;
  const uint32_t sel = hi ? 0x3232u : 0x1010u;
  asm("prmt.b32 %0, %1, %1, %2;" : "=r"(r) : "r"(w), "r"(sel));
  return r;
}

// acc[4 rows][4 pairs] = max(acc, A (x) B) over the 32 k of one staged K tile.
__device__ __forceinline__ void micro(const uint32_t* As, const uint16_t* Bs, uint32_t (&acc)[16], int lane) {
  const int ty = lane >> 2, tx = lane & 3;
#pragma unroll kMicroUnroll
  for (int k = 0; k < T; ++k) {
    const uint4 a = *reinterpret_cast<const uint4*>(As + k * T + 4 * ty);
    const uint4 b = *reinterpret_cast<const uint4*>(Bs + k * T + 8 * tx);
    const uint32_t av[4] = {a.x, a.y, a.z, a.w};
    const uint32_t bv[4] = {b.x, b.y, b.z, b.w};
#pragma unroll
    for (int r = 0; r < 4; ++r)
#pragma unroll
      for (int q = 0; q < 4; ++q) acc[r * 4 + q] = __viaddmax_s16x2(av[r], bv[q], acc[r * 4 + q]);
  }
}

constexpr int kAS = 72;                  // int16 row stride of the in-tile operand rows (64 entries + 8 pad)
constexpr int kCC = 34;                  // int16 row stride of the staged middle products
constexpr int16_t kNeg = -16000;         // masks split points outside a cell's range

// Phase-B buffers. The split terms of cell (r, c) that lie inside tiles I and J form ONE
// reduction over p' in [r+1, 32+c) (off-diagonal tiles) of AS[r][p'] + BC[c][p'], with
//   AS[r][p'] = U(I,I)[r][p']  (p' < 32; kNeg for p' <= r)  |  X[r][p'-32]  (p' >= 32; kNeg until computed)
//   BC[c][p'] = X[p'+1][c]     (p' < 32; p' = 31: the row below the tile)  |  L(J,J)[p'-32][c]  (p' >= 32)
// (X = this tile). The K = I terms pair gamma(i, 32I+p') with gamma(32I+p'+1, j), the K = J
// terms gamma(i, 32J+k) with gamma(32J+k+1, j). Every live cell of local anti-diagonal dl
// has exactly 31 + dl such terms, so chunks of 8 run warp-uniformly with no mask waste
// beyond the chunk edges; entries outside a cell's range are killed by kNeg on the A side.
// Diagonal tiles: AS[r][p' < 32] = kNeg, BC[c][32+k] = X[k+1][c] (filled as computed).
struct InTileBuf {
  int16_t as[T * kAS];
  int16_t bc[T * kAS];
  int16_t cc[T * kCC];        // C[r][c], the max over the middle tiles (phase A)
};

__device__ __forceinline__ bool pairable(const uint8_t* x, const uint8_t* pm, int n, int i, int j, int h) {
  return i < n && j < n && pm[x[i] * 4 + x[j]] && j - i - 1 >= h;
}

// Bit c of lane r: (i0 + r, j0 + c) may pair (pair set and hairpin). Four ballots give, per base,
// the columns holding it; lane r ORs the masks of the bases its own base pairs with, then clears
// the columns closer than the hairpin (about 15 instructions instead of 32 shuffles and lookups).
__device__ __forceinline__ uint32_t pair_bits(const uint8_t* x, const uint8_t* pm, int n, int i0, int j0, int h,
                                              int lane) {
  const unsigned full = 0xffffffffu;
  const int i = i0 + lane, jl = j0 + lane;
  const int xj = jl < n ? x[jl] : 4;  // 4: no base (past the end)
  const uint32_t m0 = __ballot_sync(full, xj == 0), m1 = __ballot_sync(full, xj == 1);
  const uint32_t m2 = __ballot_sync(full, xj == 2), m3 = __ballot_sync(full, xj == 3);
  if (i >= n) return 0u;
  const uint8_t* row = pm + 4 * x[i];
  uint32_t bits = (row[0] ? m0 : 0u) | (row[1] ? m1 : 0u) | (row[2] ? m2 : 0u) | (row[3] ? m3 : 0u);
  const int cmin = h + 1 + i - j0;  // j - i - 1 >= h  <=>  c >= cmin
  if (cmin > 0) bits = cmin >= 32 ? 0u : bits & ~((1u << cmin) - 1u);
  return bits;
}

__device__ __forceinline__ uint32_t opaque(uint32_t x) {
  uint32_t y;
  asm volatile("mov.b32 %0, %1;" : "=r"(y) : "r"(x));
  return y;
}
__device__ __forceinline__ uint4 lds_v4(uint32_t a) {
  uint4 v;
  asm volatile("ld.shared.v4.u32 {%0, %1, %2, %3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "r"(a));
  return v;
}
__device__ __forceinline__ int lds_s16(uint32_t a) {
  int16_t v;
  asm volatile("ld.shared.s16 %0, [%1];" : "=h"(v) : "r"(a));
  return v;
}
__device__ __forceinline__ void sts_u16(uint32_t a, int v) {
  asm volatile("st.shared.u16 [%0], %1;" ::"r"(a), "h"((int16_t)v) : "memory");
}
__device__ __forceinline__ uint32_t pk16(int lo, int hi) { return (uint32_t)(uint16_t)lo | ((uint32_t)(uint16_t)hi << 16); }

// The in-tile wavefront over staged AS / BC / CC (see InTileBuf): 63 local anti-diagonals
// (31 on a diagonal tile), one cell per lane. left = gamma(i0+r, j0-1), corner =
// gamma(i0+32, j0-1); on return AS[r][32+c] holds X[r][c] (kNeg for c <= r on diagonal
// tiles) and BC[c][...] the column entries.
__device__ __forceinline__ void wavefront(InTileBuf& B, bool diag, int left, int corner, uint32_t pairbits, int lane) {
  const unsigned full = 0xffffffffu;
  const int r = lane;
  int v = left;                                                    // X[r][c-1]
  int below_prev = __shfl_down_sync(full, left, 1);                // X[r+1][c-1]
  if (r == T - 1) below_prev = corner;
  if (diag) below_prev = 0;
  // 32-bit shared addresses, computed once (the loop is issue-bound)
  // (opaque copies: otherwise the compiler rematerialises the shared base from SR_CgaCtaId
  // inside the loop under the 128-register cap)
  const uint32_t as_s = opaque((uint32_t)__cvta_generic_to_shared(B.as) + r * (kAS * 2));
  const uint32_t bc_s = opaque((uint32_t)__cvta_generic_to_shared(B.bc));
  const uint32_t cc_s = opaque((uint32_t)__cvta_generic_to_shared(B.cc) + r * (kCC * 2));
  // first chunk: r >> 3 (off-diagonal) or 4 + (r >> 3) (diagonal), the same for the 8 lanes of
  // a quarter-warp so their 16-byte loads stay conflict-free (chunks below a lane's range are
  // masked by kNeg on the A side)
  const int qlo = diag ? 4 + (r >> 3) : (r >> 3);
  const uint32_t a_q0 = opaque(as_s + qlo * 16);
  const uint32_t b_off = qlo * 16;
  const uint32_t st_bc = (uint32_t)((diag ? T + r - 1 : r - 1) * 2);  // my X[r][c] as a B entry of column c
  // One step of the wavefront with NQ chunks (NQ covers [qlo, q_hi] of every live lane of
  // local anti-diagonal dl); the steps run in segments of constant NQ, fully unrolled.
  auto seg = [&](auto nqc, int dlA, int dlB) {
    constexpr int NQ = decltype(nqc)::value;
#pragma unroll kWaveUnroll
    for (int dl = dlA; dl <= dlB; ++dl) {
      const int c = r + dl;
      const bool live = c >= 0 && c < T;
      const int cc = live ? c : 0;
      const uint32_t bcol = opaque(bc_s + cc * (kAS * 2));
      int below = __shfl_down_sync(full, v, 1);
      if (r == T - 1) below = diag ? 0 : lds_s16(bcol + (T - 1) * 2);
      if (diag && dl == 1) below = 0;
      uint32_t a0 = 0, a1 = 0, a2 = 0, a3 = 0;  // four independent max chains (0 is neutral: gamma >= 0)
      const uint32_t pb = bcol + b_off;
#pragma unroll
      for (int t = 0; t < NQ; ++t) {
        const uint4 av = lds_v4(a_q0 + 16 * t), bv = lds_v4(pb + 16 * t);
        a0 = __viaddmax_s16x2(av.x, bv.x, a0);
        a1 = __viaddmax_s16x2(av.y, bv.y, a1);
        a2 = __viaddmax_s16x2(av.z, bv.z, a2);
        a3 = __viaddmax_s16x2(av.w, bv.w, a3);
      }
      const uint32_t acc = __vmaxs2(__vmaxs2(a0, a1), __vmaxs2(a2, a3));
      int val = max((int)(int16_t)(acc & 0xffffu), (int)(int16_t)(acc >> 16));
      val = max(val, lds_s16(cc_s + cc * 2));
      val = max(val, max(below, v));
      if ((pairbits >> cc) & 1u) val = max(val, below_prev + 1);
      if (live) {
        sts_u16(as_s + (T + c) * 2, val);
        if (r >= 1) sts_u16(bcol + st_bc, val);
        v = val;
        below_prev = below;
      }
      __syncwarp();
    }
  };
  using std::integral_constant;
  if (diag) {  // NQ = ((38 + dl) >> 3) - 3
    seg(integral_constant<int, 1>(), 1, 1);
    seg(integral_constant<int, 2>(), 2, 9);
    seg(integral_constant<int, 3>(), 10, 17);
    seg(integral_constant<int, 4>(), 18, 25);
    seg(integral_constant<int, 5>(), 26, 31);
  } else {     // NQ = ((38 + dl) >> 3) + 1
    seg(integral_constant<int, 1>(), -31, -31);
    seg(integral_constant<int, 2>(), -30, -23);
    seg(integral_constant<int, 3>(), -22, -15);
    seg(integral_constant<int, 4>(), -14, -7);
    seg(integral_constant<int, 5>(), -6, 1);
    seg(integral_constant<int, 6>(), 2, 9);
    seg(integral_constant<int, 7>(), 10, 17);
    seg(integral_constant<int, 8>(), 18, 25);
    seg(integral_constant<int, 9>(), 26, 31);
  }
}

// The same canonical traceback with the table in global memory (far from L2) and fewer
// round trips: an 8x8 window of gamma (rows i..i+7, columns j-7..j) is fetched in one round
// trip into shared memory and the unpaired / pair steps run out of it (a step moves i up or
// j down by at most one, so a window serves up to 7 steps); split points cost one round
// trip per 32 candidates. The interval stack lives in shared memory (kStk entries), deeper
// entries in global memory.
constexpr int kStk = 62;  // 62 (not 64): the batch kernel's 512-nt footprint then fits 16 CTAs per SM (228 KB)
// Trace one interval [i, j] (canonical order); the right part of every split is handed to
// push(k+1, j) and the walk continues on the left part. W x W window (rows i..i+W-1, columns
// j-W+1..j; W*W/32 values per lane per round trip); KC split candidates per lane per round trip.
template <int W, int KC, class TabT, class Push>
__device__ __forceinline__ void trace_interval(const TabT& tab, const uint8_t* x, const uint8_t* pm, int n, int h,
                                               uint8_t* db, int i, int j, int* win, int& guard, Push&& push,
                                               int lane) {
  const unsigned full = 0xffffffffu;
  int wi = -(1 << 20), wj = -(1 << 20);
  while (j - i >= 1 && --guard > 0) {
    if (!(i >= wi && i + 1 <= wi + W - 1 && j <= wj && j - 1 >= wj - W + 1)) {
      wi = i; wj = j;
      int a[W * W / 32];
#pragma unroll
      for (int q = 0; q < W * W / 32; ++q) {
        const int cell = lane + 32 * q;
        a[q] = tab.gamma(i + cell / W, j - W + 1 + cell % W);
      }
      __syncwarp();
#pragma unroll
      for (int q = 0; q < W * W / 32; ++q) win[lane + 32 * q] = a[q];
      __syncwarp();
    }
    const int* wr = win + (i - wi) * W + (j - wj + W - 1);
    const int v = wr[0], g1 = wr[W], g2 = wr[-1], g3 = wr[W - 1];
    if (v == g1) { i += 1; continue; }
    if (v == g2) { j -= 1; continue; }
    if (pairable(x, pm, n, i, j, h) && v == g3 + 1) {
      if (lane == 0) { db[i] = '('; db[j] = ')'; }
      i += 1; j -= 1;
      continue;
    }
    int kk = -1;
    for (int k0 = i + 1; kk < 0 && k0 < j; k0 += 32 * KC) {
      int s[KC];
#pragma unroll
      for (int u = 0; u < KC; ++u) {
        const int kq = k0 + lane + 32 * u;
        // gamma(i, kq) along row i from the row-major L record of row i (L(I',K)[k][c] =
        // gamma(32I'+k+1, 32K+c)): 32 consecutive k are 64 contiguous bytes instead of 32 lines
        const int gik = kq >= j ? 0 : (i >= 1 ? tab.lrow(i, kq) : tab.gamma(i, kq));
        s[u] = kq < j ? gik + tab.gamma(kq + 1, j) : -1;
      }
#pragma unroll
      for (int u = 0; u < KC; ++u) {
        const unsigned m = __ballot_sync(full, s[u] == v);
        if (kk < 0 && m) kk = k0 + 32 * u + __ffs(m) - 1;
      }
    }
    if (kk < 0) break;  // inconsistent table: cannot happen
    push(kk + 1, j);    // right part later (or elsewhere), left part now
    j = kk;
  }
}

// One warp, interval stack in shared memory (kStk entries, deeper ones in global memory).
template <int W, int KC, class TabT>
__device__ void warp_traceback_win(const TabT& tab, const uint8_t* x, const uint8_t* pm, int n, int h, uint8_t* db,
                                   int2* stk, int* win, int2* sstk, int lane) {
  for (int k = lane; k < n; k += 32) db[k] = '.';
  if (n <= 1) return;
  int sp = 1;
  if (lane == 0) sstk[0] = make_int2(0, n - 1);
  __syncwarp();
  int guard = 4 * n + 8;
  auto push = [&](int a, int b) {
    if (lane == 0) {
      if (sp < kStk) sstk[sp] = make_int2(a, b);
      else stk[sp] = make_int2(a, b);
    }
    ++sp;
    __syncwarp();
  };
  while (sp > 0 && --guard > 0) {
    --sp;
    const int2 iv = sp < kStk ? sstk[sp] : stk[sp];
    __syncwarp();
    trace_interval<W, KC>(tab, x, pm, n, h, db, iv.x, iv.y, win, guard, push, lane);
  }
}

// Work queue of intervals for the grid-wide traceback (one large problem): tickets from
// hdr[0] (head), slots published with a flag after a fence (hdr[1] = tail); hdr[2] counts
// intervals not yet finished, so a warp waiting on an unpublished slot stops when it is zero.
struct GridQueue {
  int* hdr;
  int* flag;
  int2* item;
  int cap;
};
__host__ __device__ __forceinline__ int grid_queue_cap(int64_t max_len) { return (int)max_len + 8192; }
// head, tail and outstanding count each on a 128-byte line of their own: the idle warps poll the
// count while the working warps push (tail, count) and pop (head)
constexpr int kQH = 32;             // ints per header line
constexpr int kQHdr = 3 * kQH;      // header ints before the flags

// ------------------------------------------------------------------ batch driver (one warp per problem)
// k_nuss_batch: every warp owns one problem at a time (no CTA barriers; 1-warp CTAs, as many
// per SM as shared memory allows) and sweeps its tile-diagonals itself:
//   per tile (I,J): issue the phase-B operand rows (cp.async) -> phase A over K = I+1..J-1
//   with double-buffered cp.async staging, C accumulated in registers -> C to shared ->
//   wavefront -> records.
// Records (global, one slot per warp): UTd[k][r] = gamma(32I+r, 32J+k) duplicated into both
// halves of a 32-bit word (the micro-kernel's A operand as stored, so staging is a plain
// copy), L[k][c] = gamma(32I+k+1, 32J+c) (B operand); per diagonal tile also the phase-B
// rows ASd[r][p] = U(I,I)[r][p] (kNeg for p <= r) and BCd[c][k] = L(I,I)[k][c].
constexpr int kRecW = T * T + T * T / 2;  // 32-bit words per tile record (UTd 4 KB + L 2 KB)
constexpr int kDiagW = T * T;             // 32-bit words per diagonal extra (ASd 2 KB + BCd 2 KB)
constexpr int kStageB = 6144;             // bytes per phase-A stage (A 4 KB + B 2 KB)

struct Tab2 {
  uint32_t* base;
  int nt;
  __device__ __forceinline__ uint32_t* UTd(int I, int J) const { return base + tile_id(I, J, nt) * kRecW; }
  __device__ __forceinline__ int16_t* L(int I, int J) const { return reinterpret_cast<int16_t*>(UTd(I, J) + T * T); }
  __device__ __forceinline__ int16_t* ASd(int I) const {
    return reinterpret_cast<int16_t*>(base + tiles_of(nt) * kRecW + (int64_t)I * kDiagW);
  }
  __device__ __forceinline__ int16_t* BCd(int I) const { return ASd(I) + T * T; }
  __device__ __forceinline__ int g16(int I, int J, int k, int r) const {  // UTd(I,J)[k][r] low half
    return (int)(int16_t)(__ldcg(UTd(I, J) + k * T + r) & 0xffffu);
  }
  __device__ __forceinline__ int gamma(int i, int j) const {
    if (j - i < 1) return 0;
    return g16(i / T, j / T, j % T, i % T);
  }
  // gamma(i, k), i >= 1, from the row-major L record of row i - 1 (32 consecutive k are 64
  // contiguous bytes: the traceback's split search reads rows)
  __device__ __forceinline__ int lrow(int i, int k) const {
    return (int)__ldcg(L((i - 1) / T, k / T) + ((i - 1) % T) * T + k % T);
  }
};

__device__ __forceinline__ void cp16(uint32_t s, const void* g) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(s), "l"(g) : "memory");
}
__device__ __forceinline__ void cp_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void cp_wait() { asm volatile("cp.async.wait_group %0;" ::"n"(N) : "memory"); }

__device__ __forceinline__ void stage_async(const Tab2& tab, int I, int K, int J, uint32_t st, int lane) {
  const uint32_t* a = tab.UTd(I, K);
  const int16_t* b = tab.L(K, J);
#pragma unroll
  for (int t = 0; t < 8; ++t) cp16(st + (lane + 32 * t) * 16, a + (lane + 32 * t) * 4);
#pragma unroll
  for (int t = 0; t < 4; ++t) cp16(st + 4096 + (lane + 32 * t) * 16, b + (lane + 32 * t) * 8);
}

// Phase-A operand staging by the TMA bulk-copy engine (grid sweep): a K-step's two records are
// contiguous (UTd 4 KB, L 2 KB), so one lane issues two cp.async.bulk copies that complete on the
// stage's mbarrier (expect_tx 6 KB) instead of 32 lanes issuing 12 16-byte cp.async each. One
// mbarrier per stage buffer and warp; their phase parities live in the warp's registers.
struct BulkStage {
  uint32_t bar;  // shared address of the warp's two mbarriers (8 bytes apart)
  uint32_t par;  // bit b: the parity of the phase stage b completes next
};
__device__ __forceinline__ void bulk_init(BulkStage& bs, uint32_t bar, int lane) {
  bs.bar = bar;
  bs.par = 0;
  if (lane == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(bar));
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(bar + 8));
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncwarp();
}
__device__ __forceinline__ void stage_bulk(const Tab2& tab, int I, int K, int J, uint32_t st, uint32_t bar, int lane) {
  if (lane == 0) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(6144) : "memory");
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], 4096, [%2];"
                 ::"r"(st), "l"(tab.UTd(I, K)), "r"(bar) : "memory");
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], 2048, [%2];"
                 ::"r"(st + 4096), "l"(tab.L(K, J)), "r"(bar) : "memory");
  }
}
__device__ __forceinline__ void bulk_wait(uint32_t bar, uint32_t parity) {
  asm volatile(
      "{\n\t.reg .pred done;\n\t"
      "WAIT_%=:\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 done, [%0], %1;\n\t"
      "@!done bra WAIT_%=;\n\t}\n" ::"r"(bar), "r"(parity) : "memory");
}

// Phase A over K in [K0, K1): acc (micro-kernel lane layout) = max(acc, UTd(I,K) (x) L(K,J)),
// operands staged by double-buffered cp.async (the batch kernel: with the bulk copies below
// config 5 measured 795 -> 815 ms).
__device__ __forceinline__ void products_cp(const Tab2& tab, int I, int J, int K0, int K1, uint8_t* stg,
                                            uint32_t (&acc)[16], int lane) {
  if (K0 >= K1) return;
  const uint32_t stg_s = (uint32_t)__cvta_generic_to_shared(stg);
  stage_async(tab, I, K0, J, stg_s, lane);
  cp_commit();
  for (int K = K0; K < K1; ++K) {
    const int b = (K - K0) & 1;
    if (K + 1 < K1) {
      stage_async(tab, I, K + 1, J, stg_s + (b ^ 1) * kStageB, lane);
      cp_commit();
      cp_wait<1>();
    } else {
      cp_wait<0>();
    }
    __syncwarp();
    micro(reinterpret_cast<const uint32_t*>(stg + b * kStageB),
          reinterpret_cast<const uint16_t*>(stg + b * kStageB + 4096), acc, lane);
    __syncwarp();
  }
}

// The same with the operands staged by double-buffered bulk copies (the grid sweep: config 4
// measured the same 8.67 ms either way; its records are written before a grid barrier and
// fenced for the async proxy).
__device__ __forceinline__ void products_async(const Tab2& tab, int I, int J, int K0, int K1, uint8_t* stg,
                                               uint32_t (&acc)[16], int lane, BulkStage& bs) {
  if (K0 >= K1) return;
  const uint32_t stg_s = (uint32_t)__cvta_generic_to_shared(stg);
  stage_bulk(tab, I, K0, J, stg_s, bs.bar, lane);
  for (int K = K0; K < K1; ++K) {
    const int b = (K - K0) & 1;
    if (K + 1 < K1) stage_bulk(tab, I, K + 1, J, stg_s + (b ^ 1) * kStageB, bs.bar + 8 * (b ^ 1), lane);
    bulk_wait(bs.bar + 8 * b, (bs.par >> b) & 1u);
    bs.par ^= 1u << b;
    micro(reinterpret_cast<const uint32_t*>(stg + b * kStageB),
          reinterpret_cast<const uint16_t*>(stg + b * kStageB + 4096), acc, lane);
    __syncwarp();  // every lane is done with stage b before it is refilled
  }
}

// Phase B of tile (I,J) from C in registers (acc), then its records.
__device__ void tile_finish(const Tab2& tab, int I, int J, const uint32_t (&acc)[16], int below, int left, int corner,
                            InTileBuf& B, const uint8_t* x, const uint8_t* pm, int n, int h, int lane,
                            PhaseClock& clk);

__device__ void batch_tile(const Tab2& tab, int I, int J, uint8_t* stg, InTileBuf& B, const uint8_t* x,
                           const uint8_t* pm, int n, int h, int lane, PhaseClock& clk) {
  const bool diag = I == J;
  const int r = lane;
  // scalar neighbours of the wavefront (loads in flight during phase A)
  const int below = diag ? 0 : tab.g16(I + 1, J, lane, 0);                              // X[32][c], c = lane
  const int left = diag ? 0 : tab.g16(I, J - 1, T - 1, r);                              // gamma(i0+r, j0-1)
  const int corner = (!diag && I + 1 <= J - 1) ? tab.g16(I + 1, J - 1, T - 1, 0) : 0;  // gamma(i0+32, j0-1)
  // phase A: C = max over K = I+1..J-1 of UTd(I,K) (x) L(K,J)
  uint32_t acc[16];
#pragma unroll
  for (int q = 0; q < 16; ++q) acc[q] = 0;  // gamma >= 0, so 0 is a neutral start
  products_cp(tab, I, J, I + 1, J, stg, acc, lane);
  tile_finish(tab, I, J, acc, below, left, corner, B, x, pm, n, h, lane, clk);
}

__device__ void tile_finish(const Tab2& tab, int I, int J, const uint32_t (&acc)[16], int below, int left, int corner,
                            InTileBuf& B, const uint8_t* x, const uint8_t* pm, int n, int h, int lane,
                            PhaseClock& clk) {
  const bool diag = I == J;
  const int r = lane;
  // phase B rows (the staging buffers alias them: phase A is done), C to shared (int16 [r][c])
  __syncwarp();
  clk.lap(1);
  if (!diag) {
    const uint32_t as_s = (uint32_t)__cvta_generic_to_shared(B.as + r * kAS);
    const uint32_t bc_s = (uint32_t)__cvta_generic_to_shared(B.bc + r * kAS + T);
    const int16_t* asd = tab.ASd(I) + r * T;
    const int16_t* bcd = tab.BCd(J) + r * T;
#pragma unroll
    for (int q = 0; q < 4; ++q) { cp16(as_s + 16 * q, asd + 8 * q); cp16(bc_s + 16 * q, bcd + 8 * q); }
    cp_commit();
  }
  {
    const int ty = lane >> 2, tx = lane & 3;
#pragma unroll
    for (int rr = 0; rr < 4; ++rr)
#pragma unroll
      for (int q = 0; q < 4; ++q)
        *reinterpret_cast<uint32_t*>(B.cc + (4 * ty + rr) * kCC + 8 * tx + 2 * q) = acc[rr * 4 + q];
    const uint32_t NEG2 = pk16(kNeg, kNeg);
    uint4* ar = reinterpret_cast<uint4*>(B.as + r * kAS);
    uint4* bc = reinterpret_cast<uint4*>(B.bc + r * kAS);
    const uint4 negs = make_uint4(NEG2, NEG2, NEG2, NEG2), zero = make_uint4(0, 0, 0, 0);
#pragma unroll
    for (int q = 4; q < 9; ++q) ar[q] = negs;               // X[r][*] not computed yet, pad
    if (diag) {
#pragma unroll
      for (int q = 0; q < 4; ++q) { ar[q] = negs; bc[4 + q] = zero; }
    }
#pragma unroll
    for (int q = 0; q < 3; ++q) bc[q] = zero;
    bc[3] = make_uint4(0, 0, 0, pk16(0, below));            // BC[c][31] = X[32][c]
    bc[8] = zero;
  }
  cp_wait<0>();
  const uint32_t pairbits = pair_bits(x, pm, n, I * T, J * T, h, lane);
  __syncwarp();
  clk.lap(2);
  wavefront(B, diag, left, corner, pairbits, lane);
  clk.lap(3);
  // records
  {
    const uint4* xr = reinterpret_cast<const uint4*>(B.as + r * kAS + T);
    uint4 w[4], raw[4];
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      raw[q] = w[q] = xr[q];
      if (diag) {  // entries with c <= r are gamma(i, j <= i) = 0 (held as kNeg)
        w[q].x = __vmaxs2(w[q].x, 0u); w[q].y = __vmaxs2(w[q].y, 0u);
        w[q].z = __vmaxs2(w[q].z, 0u); w[q].w = __vmaxs2(w[q].w, 0u);
      }
    }
    const uint32_t ww[16] = {w[0].x, w[0].y, w[0].z, w[0].w, w[1].x, w[1].y, w[1].z, w[1].w,
                             w[2].x, w[2].y, w[2].z, w[2].w, w[3].x, w[3].y, w[3].z, w[3].w};
    uint32_t* ut = tab.UTd(I, J);
#pragma unroll
    for (int q = 0; q < 16; ++q) {
      const uint32_t lo = ww[q] & 0xffffu, hi = ww[q] >> 16;
      ut[(2 * q) * T + r] = lo | (lo << 16);
      ut[(2 * q + 1) * T + r] = hi | (hi << 16);
    }
    int16_t* l = tab.L(I, J);
    if (r >= 1) {
      uint4* lr = reinterpret_cast<uint4*>(l + (r - 1) * T);
#pragma unroll
      for (int q = 0; q < 4; ++q) lr[q] = w[q];
    }
    l[(T - 1) * T + lane] = B.bc[lane * kAS + (T - 1)];
    if (diag) {
      uint4* asd = reinterpret_cast<uint4*>(tab.ASd(I) + r * T);
      uint4* bcd = reinterpret_cast<uint4*>(tab.BCd(I) + r * T);
      const uint4* bcr = reinterpret_cast<const uint4*>(B.bc + r * kAS + T);
#pragma unroll
      for (int q = 0; q < 4; ++q) { asd[q] = raw[q]; bcd[q] = bcr[q]; }
    }
  }
  __syncwarp();
  clk.lap(4);
}

constexpr size_t kBatchBuf = 2 * kStageB > sizeof(InTileBuf) ? 2 * kStageB : ((sizeof(InTileBuf) + 15) & ~size_t(15));
size_t batch_warp_bytes(int64_t max_len) { return kBatchBuf + ((max_len + 15) & ~int64_t(15)) + 16 + 256 + 8 * kStk; }

__global__ void __launch_bounds__(32, 16) k_nuss_batch(NussArgs A, int64_t slot_words) {
  extern __shared__ __align__(16) uint8_t smem[];
  const int lane = threadIdx.x;
  uint8_t* stg = smem;
  InTileBuf& IB = *reinterpret_cast<InTileBuf*>(smem);  // aliases the phase-A stages
  uint8_t* xs = smem + kBatchBuf;
  uint8_t* pm = xs + ((A.max_len + 15) & ~int64_t(15));
  int* win = reinterpret_cast<int*>(pm + 16);
  int2* sstk = reinterpret_cast<int2*>(pm + 16 + 256);
  if (lane < 16) pm[lane] = A.pair_mask[lane];
  Tab2 tab;
  tab.base = reinterpret_cast<uint32_t*>(A.scratch) + (int64_t)blockIdx.x * slot_words;
  const int ntm = (int)((A.max_len + T - 1) / T);
  int2* stack = reinterpret_cast<int2*>(tab.base + tiles_of(ntm) * kRecW + (int64_t)ntm * kDiagW);
  PhaseClock clk;
  clk.dbg = A.dbg;
  clk.start();
  for (;;) {
    int idx = 0;
    if (lane == 0) idx = atomicAdd(A.queue, 1);   // the next problem, longest first
    idx = __shfl_sync(0xffffffffu, idx, 0);
    if (idx >= A.n) break;
    const int64_t p = A.perm[idx];
    const int n = (int)(A.x_off[p + 1] - A.x_off[p]);
    __syncwarp();
    for (int q = lane; q < n; q += 32) xs[q] = A.x_cat[A.x_off[p] + q];
    const int nt = (n + T - 1) / T;
    tab.nt = nt;
    __syncwarp();
    clk.lap(0);
    for (int D = 0; D < nt; ++D)
      for (int t = 0; t + D < nt; ++t) batch_tile(tab, t, t + D, stg, IB, xs, pm, n, A.hairpin, lane, clk);
    clk.lap(5);
    if (lane == 0) {
      A.scores[p] = n <= 1 ? 0 : tab.gamma(0, n - 1);
      if (A.db) A.db_len[p] = n;
    }
    if (A.db) warp_traceback_win<NUSS_TBW_B, NUSS_TBK_B>(tab, xs, pm, n, A.hairpin, A.db + p * A.db_stride, stack, win, sstk, lane);
    clk.lap(6);
  }
  clk.flush(lane);
}

// ------------------------------------------------------------------ grid driver v2 (one large problem)
// k_nuss_grid2: the tile-diagonal sweep of one table over the whole grid (cooperative launch),
// on the batch kernel's records (duplicated-A UTd, L, diagonal ASd/BCd) and cp.async staging.
// Round D: phase-B warps (warp % 4 == 0, tiles spread over the SMs) add the two boundary
// K-steps I+1 and J-1 in registers, merge the interior products from global C and finish the
// tile; the other warps compute the interior K-steps of diagonal D+1 (split-K, atomicMax into
// global C). One grid-wide barrier per tile-diagonal.
__global__ void __launch_bounds__(kGridWarps * 32, 1) k_nuss_grid2(NussArgs A, int64_t p) {
  cg::grid_group grid = cg::this_grid();
  extern __shared__ __align__(16) uint8_t smem[];
  __shared__ uint8_t pm[16];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (threadIdx.x < 16) pm[threadIdx.x] = A.pair_mask[threadIdx.x];
  __syncthreads();
  uint8_t* stg = smem + warp * kBatchBuf;
  InTileBuf& IB = *reinterpret_cast<InTileBuf*>(stg);
  const int n = (int)(A.x_off[p + 1] - A.x_off[p]);
  // the sequence in shared memory (the pair tests of phase B and of the traceback's steps)
  uint8_t* x = smem + kGridWarps * kBatchBuf;
  for (int q = threadIdx.x; q < n; q += blockDim.x) x[q] = A.x_cat[A.x_off[p] + q];
  BulkStage bs;
  bulk_init(bs, (uint32_t)__cvta_generic_to_shared(x + ((A.max_len + 15) & ~int64_t(15))) + 16 * warp, lane);
  __syncthreads();
  const int nt = (n + T - 1) / T;
  Tab2 tab;
  tab.base = reinterpret_cast<uint32_t*>(A.scratch);
  tab.nt = nt;
  int* Cg = reinterpret_cast<int*>(tab.base + tiles_of(nt) * kRecW + (int64_t)nt * kDiagW);  // 2 x nt x 1024
  GridQueue Q;
  Q.hdr = Cg + 2 * (int64_t)nt * T * T;
  Q.cap = grid_queue_cap(A.max_len);
  Q.flag = Q.hdr + kQHdr;
  Q.item = reinterpret_cast<int2*>(Q.flag + Q.cap + (Q.cap & 1));
  PhaseClock clk;
  clk.dbg = A.dbg;  // DP_NUSS_TIMING: phase-B warps' per-tile phases (diagnostic)
  const int ty = lane >> 2, tx = lane & 3;
  for (int64_t q = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; q < 2 * (int64_t)nt * T * T + kQHdr + Q.cap;
       q += (int64_t)gridDim.x * blockDim.x)
    Cg[q] = 0;  // C buffers, queue counters and flags
  grid.sync();
  for (int D = 0; D < nt; ++D) {
    if (A.round_ns && blockIdx.x == 0 && threadIdx.x == 0) {
      unsigned long long t;
      asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
      A.round_ns[D] = t;
    }
    if ((warp & 3) == 0) clk.start();
    const int nT = nt - D;
    int* C = Cg + (int64_t)(D & 1) * nt * T * T;        // diagonal D (interior products already in)
    int* Cn = Cg + (int64_t)((D + 1) & 1) * nt * T * T; // diagonal D+1
    if ((warp & 3) == 0) {
      for (int64_t tt = blockIdx.x + (int64_t)gridDim.x * (warp >> 2); tt < nT;
           tt += (int64_t)gridDim.x * (kGridWarps / 4)) {
        const int t = (int)tt, I = t, J = t + D;
        const bool diag = D == 0;
        int* Ct = C + (int64_t)t * T * T;
        const int below = diag ? 0 : tab.g16(I + 1, J, lane, 0);
        const int left = diag ? 0 : tab.g16(I, J - 1, T - 1, lane);
        const int corner = (!diag && I + 1 <= J - 1) ? tab.g16(I + 1, J - 1, T - 1, 0) : 0;
        clk.start();
        uint32_t acc[16];
#pragma unroll
        for (int q = 0; q < 16; ++q) acc[q] = 0;
        if (D >= 2) products_async(tab, I, J, I + 1, I + 2, stg, acc, lane, bs);
        if (D >= 3) products_async(tab, I, J, J - 1, J, stg, acc, lane, bs);
        if (D >= 4) {  // interior K = I+2 .. J-2 from the other warps (complete at the last grid barrier)
#pragma unroll
          for (int rr = 0; rr < 4; ++rr)
#pragma unroll
            for (int q = 0; q < 4; ++q) {
              const int* cp = Ct + (4 * ty + rr) * T + 8 * tx + 2 * q;
              acc[rr * 4 + q] = __vmaxs2(acc[rr * 4 + q], pk16(__ldcg(cp), __ldcg(cp + 1)));
            }
        }
        tile_finish(tab, I, J, acc, below, left, corner, IB, x, pm, n, A.hairpin, lane, clk);
        asm volatile("fence.proxy.async.global;" ::: "memory");  // the records, before bulk copies read them
        __syncwarp();
        if (D >= 4)  // this C slot is reused by diagonal D+2
          for (int q = lane; q < T * T; q += 32) Ct[q] = 0;
        clk.lap(4);
      }
    } else if (D + 1 < nt && D >= 3) {
      // interior K-steps of diagonal D+1: tiles t' (I = t', J = t' + D + 1), K in [I+2, J-2]
      const int nT1 = nt - (D + 1), ks = D - 2;
      const int64_t total = (int64_t)nT1 * ks;
      const int64_t nwA = (int64_t)gridDim.x * (kGridWarps - kGridWarps / 4);
      const int64_t wA = (int64_t)blockIdx.x * (kGridWarps - kGridWarps / 4) + (warp - (warp >> 2) - 1);
      const int64_t per = (total + nwA - 1) / nwA;
      const int64_t b0 = wA * per, b1 = min(total, b0 + per);
      int64_t it = b0;
      while (it < b1) {
        const int t = (int)(it / ks), kk = (int)(it % ks);
        const int64_t e = min(b1, (int64_t)(t + 1) * ks);
        const int I = t, J = t + D + 1;
        uint32_t acc[16];
#pragma unroll
        for (int q = 0; q < 16; ++q) acc[q] = 0;
        products_async(tab, I, J, I + 2 + kk, I + 2 + kk + (int)(e - it), stg, acc, lane, bs);
        int* Ct = Cn + (int64_t)t * T * T;
#pragma unroll
        for (int rr = 0; rr < 4; ++rr)
#pragma unroll
          for (int q = 0; q < 4; ++q) {
            const uint32_t v = acc[rr * 4 + q];
            int* c = Ct + (4 * ty + rr) * T + 8 * tx + 2 * q;
            atomicMax(c, (int)(int16_t)(v & 0xffffu));
            atomicMax(c + 1, (int)(int16_t)(v >> 16));
          }
        it = e;
      }
    }
    grid.sync();
    if ((warp & 3) == 0) clk.lap(5);  // barrier wait of the phase-B warps
  }
  if (blockIdx.x == 0 && threadIdx.x == 0) {
    if (A.round_ns) {
      unsigned long long t;
      asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
      A.round_ns[nt] = t;
    }
    A.scores[p] = n <= 1 ? 0 : tab.gamma(0, n - 1);
    if (A.db) A.db_len[p] = n;
  }
  if (!A.db) return;
  // canonical traceback by the whole grid: intervals in a work queue (see TbQueue)
  uint8_t* db = A.db + p * A.db_stride;
  const int64_t gtid = (int64_t)blockIdx.x * blockDim.x + threadIdx.x, gthreads = (int64_t)gridDim.x * blockDim.x;
  for (int64_t q = gtid; q < n; q += gthreads) db[q] = '.';
  if (gtid == 0 && n > 1) {
    Q.item[0] = make_int2(0, n - 1);
    Q.flag[0] = 1;
    Q.hdr[kQH] = 1;      // tail
    Q.hdr[2 * kQH] = 1;  // outstanding
  }
  grid.sync();
  const unsigned full = 0xffffffffu;
  int* win = reinterpret_cast<int*>(stg);
  int guard = 4 * n + 8;
  long long tb_cyc = 0;  // DP_NUSS_ROUNDS: cycles this warp spends tracing, intervals traced
  int tb_iv = 0;
  auto push = [&](int a, int b) {
    if (lane == 0) {
      atomicAdd(&Q.hdr[2 * kQH], 1);
      const int t = atomicAdd(&Q.hdr[kQH], 1);
      if (t < Q.cap) {
        Q.item[t] = make_int2(a, b);
        __threadfence();
        atomicExch(&Q.flag[t], 1);
      }
    }
    __syncwarp();
  };
  for (;;) {
    int idx = 0;
    if (lane == 0) idx = atomicAdd(&Q.hdr[0], 1);
    idx = __shfl_sync(full, idx, 0);
    int got = 0;
    unsigned backoff = 64;  // polling back-off (ns), so idle warps do not crowd the queue's lines
    for (;;) {
      int f = 0, o = 0;
      if (lane == 0) {
        f = idx < Q.cap ? *reinterpret_cast<volatile int*>(&Q.flag[idx]) : 0;
        o = *reinterpret_cast<volatile int*>(&Q.hdr[2 * kQH]);
      }
      f = __shfl_sync(full, f, 0);
      o = __shfl_sync(full, o, 0);
      if (f) { got = 1; break; }
      if (o <= 0) break;
      __nanosleep(backoff);
      backoff = min(2 * backoff, 2048u);
    }
    if (!got) break;
    __threadfence();
    const int2 iv = __ldcg(&Q.item[idx]);
    const long long c0 = clock64();
    trace_interval<NUSS_TBW_G, NUSS_TBK_G>(tab, x, pm, n, A.hairpin, db, iv.x, iv.y, win, guard, push, lane);
    __syncwarp();
    tb_cyc += clock64() - c0;
    ++tb_iv;
    if (lane == 0) {
      __threadfence();
      atomicSub(&Q.hdr[2 * kQH], 1);
    }
  }
  if (A.round_ns) {
    if (lane == 0) {  // [nt + 2]: max cycles of one warp, [nt + 3]: sum, [nt + 4]: intervals, [nt + 5]: steps
      atomicMax(A.round_ns + nt + 2, (unsigned long long)tb_cyc);
      atomicAdd(A.round_ns + nt + 3, (unsigned long long)tb_cyc);
      atomicAdd(A.round_ns + nt + 4, (unsigned long long)tb_iv);
      atomicAdd(A.round_ns + nt + 5, (unsigned long long)(4 * n + 8 - guard));
    }
    grid.sync();
    if (gtid == 0) {
      unsigned long long t;
      asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
      A.round_ns[nt + 1] = t;
    }
  }
}

// ------------------------------------------------------------------ cluster driver
// k_nuss_cluster: one thread-block cluster of kcl CTAs per problem (mid-length problems, a few
// per batch: the regime between one warp per problem and the whole grid for one problem). The
// problem's table lives in the cluster's DISTRIBUTED SHARED MEMORY: tile (I,J) is computed by
// and stored in CTA J mod kcl (compact records: U16[c][r] = gamma(32I+r, 32J+c), column-major,
// and L16[k][c] = gamma(32I+k+1, 32J+c), row-major, 2 KB each; diagonal tiles add the phase-B
// rows ASd / BCd). Tile-diagonals are separated by cluster barriers (barrier.cluster
// arrive.release / wait.acquire: the records of diagonal D are visible cluster-wide before D+1).
// Phase A stages U16(I,K) (remote, duplicated into both s16 halves on the way) and L16(K,J)
// (local: same owner as (I,J)) through registers: the next K's DSMEM loads are in flight during
// the current micro-kernel. Phase B and the micro-kernel are the batch kernel's. A diagonal with
// at most half as many tiles as the cluster has warps splits each tile's K range over the whole
// cluster (partials merged by the tile's owner warp through DSMEM; one more cluster barrier).
constexpr int kClTile = 2 * T * T;   // int16 per tile record: U16 + L16
constexpr int kClDiag = 2 * T * T;   // int16 per diagonal extra: ASd + BCd
constexpr int kClMaxCl = 16;

struct ClArgs {
  int kcl;            // CTAs per cluster
  int warps;          // warps per CTA
  int slots, dslots;  // record slots per CTA (tiles, diagonal extras)
};

__host__ __device__ __forceinline__ int cl_slot(int I, int J, int kcl) {  // tile (I,J) in CTA J mod kcl
  const int o = J % kcl, m = J / kcl;
  return m * (o + 1) + kcl * m * (m - 1) / 2 + I;
}
inline int cl_slots(int nt, int kcl) {  // most tiles any CTA owns
  int mx = 0;
  for (int o = 0; o < kcl; ++o) {
    int c = 0;
    for (int J = o; J < nt; J += kcl) c += J + 1;
    mx = std::max(mx, c);
  }
  return mx;
}

struct ClTab {
  int16_t* base[kClMaxCl];  // each rank's record area (generic pointers into the cluster's shared memory)
  int kcl, slots;
  __device__ __forceinline__ int16_t* U16(int I, int J) const {
    return base[J % kcl] + (int64_t)cl_slot(I, J, kcl) * kClTile;
  }
  __device__ __forceinline__ int16_t* L16(int I, int J) const { return U16(I, J) + T * T; }
  __device__ __forceinline__ int16_t* ASd(int I) const { return base[I % kcl] + (int64_t)slots * kClTile + (I / kcl) * kClDiag; }
  __device__ __forceinline__ int16_t* BCd(int I) const { return ASd(I) + T * T; }
  __device__ __forceinline__ int gamma(int i, int j) const {
    if (j - i < 1) return 0;
    return U16(i / T, j / T)[(j % T) * T + (i % T)];
  }
  __device__ __forceinline__ int lrow(int i, int k) const { return L16((i - 1) / T, k / T)[((i - 1) % T) * T + k % T]; }
};

__device__ __forceinline__ void cluster_sync_all() {
  asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}

// Phase A over K in [K0, K1) from DSMEM: acc = max(acc, U(I,K) (x) L(K,J)).
__device__ __forceinline__ void cl_products(const ClTab& tab, int I, int J, int K0, int K1, uint8_t* stg,
                                            uint32_t (&acc)[16], int lane, PhaseClock& clk) {
  if (K0 >= K1) return;
  clk.lap(7);
  uint4 ra[4], rb[4];  // U16 (2 KB) and L16 (2 KB) of one K: 4 x 16 B per lane each
  auto load = [&](int K) {
    const uint4* u = reinterpret_cast<const uint4*>(tab.U16(I, K));
    const uint4* l = reinterpret_cast<const uint4*>(tab.L16(K, J));
#pragma unroll
    for (int t = 0; t < 4; ++t) { ra[t] = u[lane + 32 * t]; rb[t] = l[lane + 32 * t]; }
  };
  load(K0);
  uint32_t* As = reinterpret_cast<uint32_t*>(stg);
  uint4* Bs = reinterpret_cast<uint4*>(stg + 4096);
  for (int K = K0; K < K1; ++K) {
    __syncwarp();
#pragma unroll
    for (int t = 0; t < 4; ++t) {  // U16 word index e = lane + 32 t holds 8 int16: entries 8e .. 8e+7
      const int e = lane + 32 * t;
      const uint32_t w[4] = {ra[t].x, ra[t].y, ra[t].z, ra[t].w};
      uint4* dst = reinterpret_cast<uint4*>(As + 8 * e);
      dst[0] = make_uint4(dup16(w[0], 0), dup16(w[0], 1), dup16(w[1], 0), dup16(w[1], 1));
      dst[1] = make_uint4(dup16(w[2], 0), dup16(w[2], 1), dup16(w[3], 0), dup16(w[3], 1));
      Bs[e] = rb[t];
    }
    __syncwarp();
    clk.lap(0);  // staging (waits for this K's DSMEM loads)
    if (K + 1 < K1) load(K + 1);
    micro(As, reinterpret_cast<const uint16_t*>(Bs), acc, lane);
    clk.lap(1);  // micro-kernel
    clk.count(6);
  }
}

// Phase B of tile (I,J) from C in registers, then its records (in this CTA's shared memory).
__device__ void cl_tile_finish(const ClTab& tab, int I, int J, const uint32_t (&acc)[16], int below, int left,
                               int corner, InTileBuf& B, const uint8_t* x, const uint8_t* pm, int n, int h, int lane,
                               PhaseClock& clk) {
  const bool diag = I == J;
  const int r = lane;
  __syncwarp();
  clk.lap(7);
  if (!diag) {  // phase-B rows: AS[r][0..31] = ASd(I)[r][*], BC[r][32..63] = BCd(J)[r][*] (DSMEM)
    const uint4* asd = reinterpret_cast<const uint4*>(tab.ASd(I) + r * T);
    const uint4* bcd = reinterpret_cast<const uint4*>(tab.BCd(J) + r * T);
    uint4* ar = reinterpret_cast<uint4*>(B.as + r * kAS);
    uint4* br = reinterpret_cast<uint4*>(B.bc + r * kAS + T);
#pragma unroll
    for (int q = 0; q < 4; ++q) { ar[q] = asd[q]; br[q] = bcd[q]; }
  }
  {
    const int ty = lane >> 2, tx = lane & 3;
#pragma unroll
    for (int rr = 0; rr < 4; ++rr)
#pragma unroll
      for (int q = 0; q < 4; ++q)
        *reinterpret_cast<uint32_t*>(B.cc + (4 * ty + rr) * kCC + 8 * tx + 2 * q) = acc[rr * 4 + q];
    const uint32_t NEG2 = pk16(kNeg, kNeg);
    uint4* ar = reinterpret_cast<uint4*>(B.as + r * kAS);
    uint4* bc = reinterpret_cast<uint4*>(B.bc + r * kAS);
    const uint4 negs = make_uint4(NEG2, NEG2, NEG2, NEG2), zero = make_uint4(0, 0, 0, 0);
#pragma unroll
    for (int q = 4; q < 9; ++q) ar[q] = negs;
    if (diag) {
#pragma unroll
      for (int q = 0; q < 4; ++q) { ar[q] = negs; bc[4 + q] = zero; }
    }
#pragma unroll
    for (int q = 0; q < 3; ++q) bc[q] = zero;
    bc[3] = make_uint4(0, 0, 0, pk16(0, below));
    bc[8] = zero;
  }
  const uint32_t pairbits = pair_bits(x, pm, n, I * T, J * T, h, lane);
  __syncwarp();
  clk.lap(2);  // phase-B setup (DSMEM rows, C, pair bits)
  wavefront(B, diag, left, corner, pairbits, lane);
  clk.lap(3);  // wavefront
  // records: U16[c][r] (column-major) and L16[k][c] (row-major; row 31 = the row below)
  {
    const uint4* xr = reinterpret_cast<const uint4*>(B.as + r * kAS + T);
    uint4 w[4], raw[4];
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      raw[q] = w[q] = xr[q];
      if (diag) {
        w[q].x = __vmaxs2(w[q].x, 0u); w[q].y = __vmaxs2(w[q].y, 0u);
        w[q].z = __vmaxs2(w[q].z, 0u); w[q].w = __vmaxs2(w[q].w, 0u);
      }
    }
    int16_t* u = tab.U16(I, J);
    const uint32_t ww[16] = {w[0].x, w[0].y, w[0].z, w[0].w, w[1].x, w[1].y, w[1].z, w[1].w,
                             w[2].x, w[2].y, w[2].z, w[2].w, w[3].x, w[3].y, w[3].z, w[3].w};
#pragma unroll
    for (int q = 0; q < 16; ++q) {
      u[(2 * q) * T + r] = (int16_t)(ww[q] & 0xffffu);
      u[(2 * q + 1) * T + r] = (int16_t)(ww[q] >> 16);
    }
    int16_t* l = tab.L16(I, J);
    if (r >= 1) {
      uint4* lr = reinterpret_cast<uint4*>(l + (r - 1) * T);
#pragma unroll
      for (int q = 0; q < 4; ++q) lr[q] = w[q];
    }
    l[(T - 1) * T + lane] = B.bc[lane * kAS + (T - 1)];
    if (diag) {
      uint4* asd = reinterpret_cast<uint4*>(tab.ASd(I) + r * T);
      uint4* bcd = reinterpret_cast<uint4*>(tab.BCd(I) + r * T);
      const uint4* bcr = reinterpret_cast<const uint4*>(B.bc + r * kAS + T);
#pragma unroll
      for (int q = 0; q < 4; ++q) { asd[q] = raw[q]; bcd[q] = bcr[q]; }
    }
  }
  __syncwarp();
  clk.lap(4);  // records
  clk.count(5);
}

__global__ void k_nuss_cluster(NussArgs A, ClArgs C) {
  extern __shared__ __align__(16) uint8_t smem[];
  cg::cluster_group cluster = cg::this_cluster();
  const int rank = (int)cluster.block_rank(), kcl = C.kcl;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31, W = C.warps;
  int16_t* rec = reinterpret_cast<int16_t*>(smem);
  uint8_t* xs = smem + ((int64_t)C.slots * kClTile + (int64_t)C.dslots * kClDiag) * 2;
  uint8_t* pm = xs + ((A.max_len + 15) & ~int64_t(15));
  uint8_t* wbuf = pm + 16 + warp * kBatchBuf;
  int* win = reinterpret_cast<int*>(pm + 16 + W * kBatchBuf);
  int2* sstk = reinterpret_cast<int2*>(win + 64);
  if (threadIdx.x < 16) pm[threadIdx.x] = A.pair_mask[threadIdx.x];
  ClTab tab;
  tab.kcl = kcl;
  tab.slots = C.slots;
  for (int q = 0; q < kcl; ++q) tab.base[q] = cluster.map_shared_rank(rec, q);
  InTileBuf& IB = *reinterpret_cast<InTileBuf*>(wbuf);
  PhaseClock clk;  // DP_NUSS_TIMING (diagnostic): 0 staging, 1 micro, 2 phase-B setup, 3 wavefront,
  clk.dbg = A.dbg; // 4 records, 5 tiles, 6 K-steps
  clk.start();
  const int64_t nclusters = gridDim.x / kcl, cid = blockIdx.x / kcl;
  int2* gstack = reinterpret_cast<int2*>(A.scratch) + cid * (2 * A.max_len + 8);
  for (int64_t p = cid; p < A.n; p += nclusters) {
    const int n = (int)(A.x_off[p + 1] - A.x_off[p]);
    const int nt = (n + T - 1) / T;
    cluster_sync_all();  // the previous problem's traceback no longer reads any rank's records
    for (int q = threadIdx.x; q < n; q += blockDim.x) xs[q] = A.x_cat[A.x_off[p] + q];
    __syncthreads();
    for (int D = 0; D < nt; ++D) {
      if (A.round_ns && cid == 0 && rank == 0 && threadIdx.x == 0) {  // DP_NUSS_ROUNDS (diagnostic)
        unsigned long long tm;
        asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(tm));
        A.round_ns[2 * D] = tm;
      }
      // this CTA's tiles of diagonal D: J = I + D with J mod kcl == rank, one warp each
      const int I0 = ((rank - D) % kcl + kcl) % kcl;
      const int TD = nt - D, NW = kcl * W;
      if (TD * 2 > NW) {
        // many tiles: each tile on one warp of its owner CTA (at most W per owner)
        for (int I = I0 + kcl * warp; I < TD; I += kcl * W) {
          const int J = I + D;
          const bool diag = D == 0;
          const int below = diag ? 0 : tab.U16(I + 1, J)[lane * T + 0];           // X[32][c], c = lane
          const int left = diag ? 0 : tab.U16(I, J - 1)[(T - 1) * T + lane];      // gamma(32I + r, 32J - 1)
          const int corner = (!diag && I + 1 <= J - 1) ? tab.U16(I + 1, J - 1)[(T - 1) * T] : 0;
          uint32_t acc[16];
#pragma unroll
          for (int q = 0; q < 16; ++q) acc[q] = 0;
          cl_products(tab, I, J, I + 1, J, wbuf, acc, lane, clk);
          cl_tile_finish(tab, I, J, acc, below, left, corner, IB, xs, pm, n, A.hairpin, lane, clk);
        }
      } else {
        // few tiles: split-K over the whole cluster. Tile t's leader is warp t / kcl of its owner
        // CTA (part 0 of its K range); the other warps are helpers, helper h taking part
        // 1 + h / TD of tile h mod TD. Partial products stay in the computing warp's buffer; after
        // a cluster barrier each leader merges its helpers' partials through DSMEM and finishes the
        // tile (a leader's buffer only ever holds its own tile's part: no leader reads another's).
        int H = 0, h = -1;  // helpers in total, this warp's helper index
        for (int r2 = 0; r2 < kcl; ++r2) {
          const int i0 = ((r2 - D) % kcl + kcl) % kcl;
          const int lead = i0 < TD ? (TD - i0 + kcl - 1) / kcl : 0;  // leaders in CTA r2 (<= W / 2)
          if (r2 == rank && warp >= lead) h = H + (warp - lead);
          H += W - lead;
        }
        const bool leader = h < 0;
        const int t = leader ? I0 + kcl * warp : h % TD;  // my tile
        const int part = leader ? 0 : 1 + h / TD;
        const int parts = 1 + (H > t ? (H - 1 - t) / TD + 1 : 0);
        const int I = t, J = t + D, nk = J - I - 1;
        uint32_t acc[16];
#pragma unroll
        for (int q = 0; q < 16; ++q) acc[q] = 0;
        cl_products(tab, I, J, I + 1 + nk * part / parts, I + 1 + nk * (part + 1) / parts, wbuf, acc, lane, clk);
        __syncwarp();
        uint32_t* pw = reinterpret_cast<uint32_t*>(wbuf);  // the partial: word q * 32 + lane
        if (!leader) {
#pragma unroll
          for (int q = 0; q < 16; ++q) pw[q * 32 + lane] = acc[q];
        }
        cluster_sync_all();  // every partial of the diagonal written
        if (A.round_ns && cid == 0 && rank == 0 && threadIdx.x == 0) {
          unsigned long long tm;
          asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(tm));
          A.round_ns[2 * D + 1] = tm;
        }
        if (leader) {
          for (int pp = 1; pp < parts; ++pp) {
            const int hh = t + TD * (pp - 1);  // helper index of part pp
            int rq = 0, wq = 0, acc_h = 0;     // its CTA and warp
            for (int r2 = 0; r2 < kcl; ++r2) {
              const int i0 = ((r2 - D) % kcl + kcl) % kcl;
              const int lead = i0 < TD ? (TD - i0 + kcl - 1) / kcl : 0;
              if (hh < acc_h + (W - lead)) { rq = r2; wq = lead + (hh - acc_h); break; }
              acc_h += W - lead;
            }
            const uint32_t* rp = cluster.map_shared_rank(reinterpret_cast<uint32_t*>(pm + 16 + wq * kBatchBuf), rq);
#pragma unroll
            for (int q = 0; q < 16; ++q) acc[q] = __vmaxs2(acc[q], rp[q * 32 + lane]);
          }
          const bool diag = D == 0;
          const int below = diag ? 0 : tab.U16(I + 1, J)[lane * T + 0];
          const int left = diag ? 0 : tab.U16(I, J - 1)[(T - 1) * T + lane];
          const int corner = (!diag && I + 1 <= J - 1) ? tab.U16(I + 1, J - 1)[(T - 1) * T] : 0;
          cl_tile_finish(tab, I, J, acc, below, left, corner, IB, xs, pm, n, A.hairpin, lane, clk);
        }
      }
      cluster_sync_all();  // diagonal D's records visible to every rank
    }
    if (rank == 0 && threadIdx.x == 0) {
      A.scores[p] = n <= 1 ? 0 : tab.gamma(0, n - 1);
      if (A.db) A.db_len[p] = n;
    }
    if (A.db && rank == 0 && warp == 0)
      warp_traceback_win<NUSS_TBW_B, NUSS_TBK_B>(tab, xs, pm, n, A.hairpin, A.db + p * A.db_stride, gstack, win, sstk,
                                                 lane);
  }
  cluster_sync_all();  // no rank exits while rank 0 may still read its records
}

size_t cl_smem_bytes(int64_t max_len, int slots, int dslots, int warps) {
  return ((size_t)slots * kClTile + (size_t)dslots * kClDiag) * 2 + ((max_len + 15) & ~int64_t(15)) + 16 +
         (size_t)warps * kBatchBuf + 256 + 8 * kStk;
}

// the cluster configuration for problems of max_len: the smallest kcl whose per-CTA records and
// at least two warps' buffers fit; 0 if none
ClArgs cl_config(int64_t max_len, int smem_optin) {
  ClArgs c{};
  const int nt = (int)((max_len + T - 1) / T);
  for (int kcl : {2, 4, 8, 16}) {
    const int slots = cl_slots(nt, kcl), dslots = (nt + kcl - 1) / kcl;
    for (int w = 4; w >= 2; --w)
      if (cl_smem_bytes(max_len, slots, dslots, w) <= (size_t)smem_optin) {
        c.kcl = kcl; c.warps = w; c.slots = slots; c.dslots = dslots;
        return c;
      }
  }
  return c;
}

int num_sms_t(int device) {
  int v = 0;
  cudaDeviceGetAttribute(&v, cudaDevAttrMultiProcessorCount, device);
  return v > 0 ? v : 148;
}

int64_t batch_slot_words(int64_t max_len) {
  const int nt = (int)((max_len + T - 1) / T);
  return tiles_of(nt) * kRecW + (int64_t)nt * kDiagW + 2 * (2 * max_len + 8);
}

int batch_ctas_per_sm(int64_t max_len) {
  const size_t smem = batch_warp_bytes(max_len);
  cudaFuncSetAttribute(k_nuss_batch, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  cudaFuncSetAttribute(k_nuss_batch, cudaFuncAttributePreferredSharedMemoryCarveout, 100);
  int per_sm = 0;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k_nuss_batch, 32, smem);
  return per_sm > 0 ? per_sm : 1;
}

// ------------------------------------------------------------------ cost-sorted work queue (A7)
// the batch warps take problems from an atomic counter in
// decreasing length (cost ~ n^3), so the last problems handed out are the cheapest and the
// warps finish together. The order is a device counting sort by length: histogram, a descending
// exclusive scan (one CTA), a scatter (ties in any order: outputs are written by problem id).
__global__ void k_len_hist(const int64_t* off, int64_t n, int* hist, int64_t max_len) {
  for (int64_t p = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; p < n; p += (int64_t)gridDim.x * blockDim.x)
    atomicAdd(&hist[min(off[p + 1] - off[p], max_len)], 1);
}

__global__ void k_len_scan(int* hist, int64_t max_len) {  // one CTA: hist[l] <- sum of hist[l' > l]
  __shared__ int part[1024];
  const int nb = (int)max_len + 1, t = threadIdx.x;
  const int per = (nb + 1023) / 1024;
  // thread t owns lengths (in descending order) d in [t per, (t+1) per), d = max_len - l
  int sum = 0;
  for (int d = t * per; d < min(nb, (t + 1) * per); ++d) sum += hist[(int)max_len - d];
  part[t] = sum;
  __syncthreads();
  for (int o = 1; o < 1024; o <<= 1) {
    const int v = t >= o ? part[t - o] : 0;
    __syncthreads();
    part[t] += v;
    __syncthreads();
  }
  int run = t > 0 ? part[t - 1] : 0;
  for (int d = t * per; d < min(nb, (t + 1) * per); ++d) {
    const int l = (int)max_len - d, c = hist[l];
    hist[l] = run;
    run += c;
  }
}

__global__ void k_len_scatter(const int64_t* off, int64_t n, int* hist, int* perm, int64_t max_len) {
  for (int64_t p = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; p < n; p += (int64_t)gridDim.x * blockDim.x)
    perm[atomicAdd(&hist[min(off[p + 1] - off[p], max_len)], 1)] = (int)p;
}

}  // namespace

// NEXT 4: a few mid-length problems, one cluster each (see k_nuss_cluster)
bool nuss_cluster_supported(int64_t max_len, int64_t n, int device) {
  if (max_len <= 128 || max_len > 1024 || n > 64) return false;
  int optin = 0;
  cudaDeviceGetAttribute(&optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, device);
  return cl_config(max_len, optin).kcl > 0;
}

int64_t nuss_cluster_scratch_bytes(int64_t max_len, int64_t n) { return n * (2 * max_len + 8) * 8 + 256; }

cudaError_t nuss_cluster_solve(const NussArgs& A, cudaStream_t s, int64_t* launches) {
  if (A.n == 0) return cudaSuccess;
  int dev = 0, optin = 0;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev);
  const ClArgs C = cl_config(A.max_len, optin);
  if (C.kcl == 0) return cudaErrorInvalidValue;
  const size_t smem = cl_smem_bytes(A.max_len, C.slots, C.dslots, C.warps);
  cudaError_t e = cudaFuncSetAttribute(k_nuss_cluster, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e == cudaSuccess && C.kcl > 8) e = cudaFuncSetAttribute(k_nuss_cluster, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
  if (e != cudaSuccess) return e;
  cudaLaunchConfig_t cfg = {};
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeClusterDimension;
  attr[0].val.clusterDim.x = C.kcl;
  attr[0].val.clusterDim.y = 1;
  attr[0].val.clusterDim.z = 1;
  cfg.blockDim = dim3(32 * C.warps, 1, 1);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = s;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  cfg.gridDim = dim3(C.kcl, 1, 1);
  int clusters = 0;
  e = cudaOccupancyMaxActiveClusters(&clusters, k_nuss_cluster, &cfg);
  if (e != cudaSuccess) return e;
  if (clusters < 1) return cudaErrorInvalidConfiguration;
  cfg.gridDim = dim3((unsigned)(std::min<int64_t>(A.n, clusters) * C.kcl), 1, 1);
  ++*launches;
  return cudaLaunchKernelEx(&cfg, k_nuss_cluster, A, C);
}

bool nuss_tiled_supported(int64_t max_len) { return max_len <= 65536; }

int64_t nuss_tiled_scratch_bytes(int64_t max_len, int64_t n, int device) {
  const int nt = (int)((max_len + T - 1) / T);
  if (n == 1 && max_len > kGridMin)
    return (tiles_of(nt) * kRecW + (int64_t)nt * kDiagW + 2 * (int64_t)nt * T * T) * 4 +
           (kQHdr + 3 * (int64_t)grid_queue_cap(max_len) + 2) * 4 + 256;
  const int64_t grid = std::min<int64_t>(n, (int64_t)batch_ctas_per_sm(max_len) * num_sms_t(device));
  // + the work queue: counter, length histogram, permutation
  return grid * batch_slot_words(max_len) * 4 + 256 + 16 + (max_len + 1) * 4 + n * 4 + 256;
}

cudaError_t nuss_tiled_solve(const NussArgs& A, cudaStream_t s, int64_t* launches) {
  if (A.n == 0) return cudaSuccess;
  int dev = 0;
  cudaGetDevice(&dev);
  const int sms = num_sms_t(dev);
  if (A.n == 1 && A.max_len > kGridMin) {
    const size_t smem = kGridWarps * kBatchBuf + ((A.max_len + 15) & ~int64_t(15)) + 16 * kGridWarps;
    cudaError_t e = cudaFuncSetAttribute(k_nuss_grid2, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    int per_sm = 0;
    e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k_nuss_grid2, kGridWarps * 32, smem);
    if (e != cudaSuccess) return e;
    if (per_sm < 1) return cudaErrorInvalidConfiguration;
    NussArgs a2 = A;
    int64_t p = 0;
    void* args[2] = {&a2, &p};
    ++*launches;
    return cudaLaunchCooperativeKernel((void*)k_nuss_grid2, sms, kGridWarps * 32, args, smem, s);
  }
  if (A.max_len > 4096) return cudaErrorInvalidValue;  // batch path keeps the sequence in shared memory
  const int per_sm = batch_ctas_per_sm(A.max_len);
  const int64_t grid = std::min<int64_t>(A.n, (int64_t)per_sm * sms);
  const int64_t slot_words = batch_slot_words(A.max_len);
  // work queue after the slots: [counter, pad][hist: max_len + 1][perm: n]
  NussArgs a2 = A;
  int* q = reinterpret_cast<int*>(reinterpret_cast<uint8_t*>(A.scratch) + ((grid * slot_words * 4 + 255) & ~int64_t(255)));
  a2.queue = q;
  int* hist = q + 4;
  int* perm = hist + ((A.max_len + 1 + 3) & ~int64_t(3));
  a2.perm = perm;
  cudaError_t e = cudaMemsetAsync(q, 0, (size_t)(4 + A.max_len + 1) * 4, s);
  if (e != cudaSuccess) return e;
  const unsigned gs = (unsigned)std::min<int64_t>((A.n + 255) / 256, (int64_t)sms * 8);
  k_len_hist<<<gs, 256, 0, s>>>(A.x_off, A.n, hist, A.max_len);
  k_len_scan<<<1, 1024, 0, s>>>(hist, A.max_len);
  k_len_scatter<<<gs, 256, 0, s>>>(A.x_off, A.n, hist, perm, A.max_len);
  *launches += 4;
  k_nuss_batch<<<(unsigned)grid, 32, batch_warp_bytes(A.max_len), s>>>(a2, slot_words);
  return cudaGetLastError();
}

}  // namespace dpk

