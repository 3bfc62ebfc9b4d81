// Nussinov interval DP on the hyperplanes of the derived schedule
// S(i,j) = -i + j (partition d = j - i):
//   gamma(i,j) = max{ gamma(i+1,j), gamma(i,j-1), gamma(i+1,j-1) + 1 [pair, j-i-1 >= h],
//                     max_{i<k<j} gamma(i,k) + gamma(k+1,j) }.
// The recurrence is not in PAPER.md (RNA folding is Further Work, L585–L589);
// the definition follows the paper's ref [3] (DESIGN.md R-NUSS).
//
// Table layout (int16, scores <= n/2): two triangular copies so that both
// operand streams of a split term are contiguous in k:
//   U[i][k] = gamma(i, k),   k = i .. n-1      (row i)
//   L[j][k] = gamma(k+1, j), k = 0 .. j-1      (row j)
// split(i,j) = max_k U[i][k] + L[j][k] over i < k < j.
// Cells of one partition are independent (eq.2), so a partition is computed
// by all threads of the CTA (or grid) and closed by one barrier (Fig.8).
// Each cell is reduced by a power-of-two group of lanes (k strided over the
// group, then __shfl_xor_sync), sized to the partition's cell count.
#include <algorithm>
#include <cstdint>
#include <cooperative_groups.h>
#include <cuda_runtime.h>

#include "dp_internal.h"

namespace cg = cooperative_groups;

namespace dpk {
namespace {

constexpr int kNussThreads = 512;
constexpr int64_t kSmemMaxN = 340;  // 2 n^2 bytes of int16 table <= 227 KiB
constexpr int64_t kSmemStackN = 256;  // the traceback stack (4 n + 8 ints) also in shared memory up to here

__host__ __device__ __forceinline__ int64_t ustart(int64_t i, int64_t n) { return i * n - (i * (i - 1)) / 2; }
__host__ __device__ __forceinline__ int64_t lstart(int64_t j) { return (j * (j - 1)) / 2; }
// n(n+1)/2 (U) + n(n-1)/2 (L), rounded to 8 elements so what follows stays 16-byte aligned
__host__ __device__ __forceinline__ int64_t table_elems(int64_t n) { return (n * n + 7) & ~int64_t(7); }

// Evaluate the cells of partition d assigned to this thread. `tid`/`nthr`
// span the CTA (or the whole grid).
__device__ __forceinline__ void nuss_partition(int16_t* U, int16_t* L, const uint8_t* x, int n, int d,
                                               const uint8_t* pm, int h, int64_t tid64, int64_t nthr64) {
  const int ncells = n - d;
  // group size G = 2^lg: power of two <= 32, about nthr / ncells lanes per cell, no more than the
  // split count (32-bit index math, shifts: this runs once per partition per thread)
  const int tid = (int)tid64, nthr = (int)nthr64;
  int lg = 0;
  while (lg < 5 && (2 << lg) * ncells <= nthr && (2 << lg) <= max(1, d - 1)) ++lg;
  const int G = 1 << lg;
  const int ngroups = nthr >> lg;
  const int q = tid & (G - 1);
  const int grp = tid >> lg;
  // every group runs the same number of iterations so the shuffles stay converged
  const int iters = (ncells + ngroups - 1) / ngroups;
  for (int it = 0; it < iters; ++it) {
    const int cidx = grp + it * ngroups;
    const bool live = cidx < ncells;
    const int i = live ? cidx : 0;
    const int j = i + d;
    int best = 0;
    if (live) {
      const int16_t* Ui = U + ustart(i, n) - i;  // Ui[k] = gamma(i, k)
      const int16_t* Lj = L + lstart(j);
      for (int k = i + 1 + q; k < j; k += G) best = max(best, (int)Ui[k] + (int)Lj[k]);
    }
    const unsigned mask = 0xffffffffu;
    if (G > 1) {
      for (int o = G / 2; o > 0; o >>= 1) best = max(best, __shfl_xor_sync(mask, best, o, G));
    }
    if (live && q == 0) {
      const int16_t* Ui = U + ustart(i, n);
      const int16_t* Ui1 = U + ustart(i + 1, n);
      int v = best;
      v = max(v, (int)Ui1[j - (i + 1)]);               // gamma(i+1, j)
      v = max(v, (int)Ui[j - 1 - i]);                  // gamma(i, j-1)
      if (pm[x[i] * 4 + x[j]] && d - 1 >= h) {
        const int inner = (d >= 2) ? (int)Ui1[j - 1 - (i + 1)] : 0;  // gamma(i+1, j-1), empty -> 0
        v = max(v, inner + 1);
      }
      U[ustart(i, n) + d] = (int16_t)v;
      if (i >= 1) L[lstart(j) + (i - 1)] = (int16_t)v;
    }
  }
}

__device__ void nuss_init(int16_t* U, int16_t* L, int n, int64_t tid, int64_t nthr) {
  // diagonal d = 0: gamma(i,i) = 0 in U; L[j][j-1] = gamma(j,j) = 0
  for (int64_t i = tid; i < n; i += nthr) {
    U[ustart(i, n)] = 0;
    if (i >= 1) L[lstart(i) + i - 1] = 0;
  }
}

// Canonical traceback (DESIGN.md R-TB-NUSS): Durbin order, smallest split k.
// One warp: lane 0 owns the explicit stack (global scratch, L1/L2-resident);
// the split search is spread over the 32 lanes and the smallest matching k is
// taken with a ballot, so a step costs ceil((j-i-1)/32) table reads per lane
// instead of j-i-1 serial ones.
__device__ void nuss_traceback_warp(const int16_t* U, const int16_t* L, const uint8_t* x, int n, const uint8_t* pm,
                                    int h, uint8_t* db, int* stack) {
  const int lane = threadIdx.x & 31;
  for (int k = lane; k < n; k += 32) db[k] = '.';
  if (n <= 1) return;
  __syncwarp();
  auto gam = [&](int i, int j) -> int { return (j - i < 1) ? 0 : (int)U[ustart(i, n) + (j - i)]; };
  int sp = 0;  // identical in every lane
  if (lane == 0) { stack[0] = 0; stack[1] = n - 1; }
  sp = 2;
  int guard = 4 * n + 8;
  while (sp > 0 && --guard > 0) {
    __syncwarp();
    const int j = stack[sp - 1], i = stack[sp - 2];
    sp -= 2;
    if (j - i < 1) continue;
    const int v = gam(i, j);
    int ni0 = -1, nj0 = 0, ni1 = -1, nj1 = 0;  // up to two intervals to push (second on top)
    if (v == gam(i + 1, j)) {
      ni0 = i + 1; nj0 = j;
    } else if (v == gam(i, j - 1)) {
      ni0 = i; nj0 = j - 1;
    } else if (pm[x[i] * 4 + x[j]] && j - i - 1 >= h && v == gam(i + 1, j - 1) + 1) {
      if (lane == 0) { db[i] = '('; db[j] = ')'; }
      ni0 = i + 1; nj0 = j - 1;
    } else {
      const int16_t* Ui = U + ustart(i, n);
      const int16_t* Lj = L + lstart(j);
      for (int k0 = i + 1; k0 < j; k0 += 32) {
        const int k = k0 + lane;
        const unsigned hit = __ballot_sync(0xffffffffu, k < j && v == (int)Ui[k - i] + (int)Lj[k]);
        if (hit) {
          const int kk = k0 + __ffs(hit) - 1;
          ni0 = kk + 1; nj0 = j; ni1 = i; nj1 = kk;
          break;
        }
      }
    }
    __syncwarp();
    if (ni0 >= 0) {
      if (lane == 0) { stack[sp] = ni0; stack[sp + 1] = nj0; }
      sp += 2;
    }
    if (ni1 >= 0) {
      if (lane == 0) { stack[sp] = ni1; stack[sp + 1] = nj1; }
      sp += 2;
    }
  }
}

// One CTA per problem (persistent over the batch). The table lives in shared
// memory when it fits (SMEM=true) or in this CTA's slice of a global scratch
// that stays L2-resident (SMEM=false).
template <bool SMEM>
__global__ void __launch_bounds__(kNussThreads) k_nuss_cta(NussArgs A, int64_t slice_elems) {
  extern __shared__ __align__(16) uint8_t smem[];
  __shared__ uint8_t pm[16];
  if (threadIdx.x < 16) pm[threadIdx.x] = A.pair_mask[threadIdx.x];
  uint8_t* xs = smem;  // sequence bytes
  int16_t* tab;
  if (SMEM) tab = reinterpret_cast<int16_t*>(smem + ((A.max_len + 15) & ~15));
  else tab = reinterpret_cast<int16_t*>(A.scratch) + (int64_t)blockIdx.x * slice_elems;
  int* stack = reinterpret_cast<int*>(reinterpret_cast<int16_t*>(A.scratch) + (int64_t)gridDim.x * (SMEM ? 0 : slice_elems)) +
               (int64_t)blockIdx.x * (4 * A.max_len + 8);
  if (SMEM && A.max_len <= kSmemStackN)  // the traceback's interval stack next to the table
    stack = reinterpret_cast<int*>(tab + table_elems(A.max_len));
  for (int64_t p = blockIdx.x; p < A.n; p += gridDim.x) {
    const uint8_t* xg = A.x_cat + A.x_off[p];
    const int n = (int)(A.x_off[p + 1] - A.x_off[p]);
    __syncthreads();
    for (int q = threadIdx.x; q < n; q += blockDim.x) xs[q] = xg[q];
    int16_t* U = tab;
    int16_t* L = tab + (int64_t)n * (n + 1) / 2;
    nuss_init(U, L, n, threadIdx.x, blockDim.x);
    __syncthreads();
    for (int d = 1; d < n; ++d) {
      nuss_partition(U, L, xs, n, d, pm, A.hairpin, threadIdx.x, blockDim.x);
      __syncthreads();
    }
    if (threadIdx.x == 0) A.scores[p] = n <= 1 ? 0 : (int)U[ustart(0, n) + n - 1];
    if (A.db && threadIdx.x < 32) {
      nuss_traceback_warp(U, L, xs, n, pm, A.hairpin, A.db + p * A.db_stride, stack);
      if (threadIdx.x == 0) A.db_len[p] = n;
    }
  }
}

// ------------------------------------------------------------------ short problems, latency-bound
// k_nuss_small (one 64-nt RNA is 63 dependent partitions, a latency problem):
// one small CTA per problem, the whole table in shared memory, one barrier per partition (Fig.8's
// `sync`, L251–L253), thread r owning the cells of rows r, r + 64; the traceback from the same
// shared table. Measured (config 1, clock64): ~600 cycles per partition, set by each cell's
// serial chain of dependent shared-memory round trips (the loop and barrier alone: 28 cycles),
// 13k cycles of traceback. Both copies are full squares
// of row stride W (W / 8 odd: rows 8 lanes apart fall on distinct bank quads):
//   U[i][k] = gamma(i, k) (k >= i), L[j][k] = gamma(k+1, j) (k < j), L[j][j] = 0,
// every other entry (and every entry not yet computed) kNeg. Then for a cell of partition d
//   max_{i <= k <= j} U[i][k] + L[j][k] = max(gamma(i+1, j), gamma(i, j-1), split terms)
// (k = i: the "i unpaired" term; k = j-1: "j unpaired"; k = j and k < i: kNeg), so a cell is one
// s16x2 max-plus reduction over the aligned 8-wide chunks covering [i, j] plus the pair term.
// Entries read but written in the same partition (U[i][j], L[j][i-1]) are this cell's own and
// pair with kNeg; they are written after the cell's reduction.
constexpr int kSmallMaxN = 128;
constexpr int kSmallThreads = 64;  // n <= 64: one cell per thread per partition (32 / 64 / 128 threads:
                                   // 45.1k / 41.5k / 41.5k cycles of fill for config 1)
constexpr int16_t kSNeg = -16000;

__host__ __device__ __forceinline__ int small_w(int64_t max_len) { return 8 * ((int)((max_len + 7) / 8) | 1); }
size_t small_smem_bytes(int64_t max_len) {
  const int w = small_w(max_len);
  return (size_t)2 * max_len * w * 2 + 128 + 16 + 128 + (size_t)(4 * max_len + 8) * 4;
}

__global__ void __launch_bounds__(kSmallThreads) k_nuss_small(NussArgs A) {
  extern __shared__ __align__(16) uint8_t smem[];
  const int W = small_w(A.max_len);
  int16_t* U = reinterpret_cast<int16_t*>(smem);
  int16_t* L = U + A.max_len * W;
  uint8_t* xs = reinterpret_cast<uint8_t*>(L + A.max_len * W);
  uint8_t* pm = xs + 128;
  uint8_t* prow = pm + 16;
  int* stack = reinterpret_cast<int*>(prow + 128);
  const int tid = threadIdx.x, lane = tid & 31;
  if (tid < 16) pm[tid] = A.pair_mask[tid];
  const uint32_t NEG2 = (uint32_t)(uint16_t)kSNeg * 0x10001u;
  long long t0 = A.dbg ? clock64() : 0;  // DP_NUSS_TIMING: thread 0's cycles in setup / fill / traceback
  auto lap = [&](int k) {
    if (A.dbg && tid == 0) {
      const long long t = clock64();
      atomicAdd(A.dbg + k, (unsigned long long)(t - t0));
      t0 = t;
    }
  };
  for (int64_t p = blockIdx.x; p < A.n; p += gridDim.x) {
    const int n = (int)(A.x_off[p + 1] - A.x_off[p]);
    __syncthreads();
    for (int q = tid; q < n; q += blockDim.x) xs[q] = A.x_cat[A.x_off[p] + q];
    for (int r = tid >> 5; r < n; r += kSmallThreads / 32) {  // a warp per row, two entries per word
      uint32_t* ur = reinterpret_cast<uint32_t*>(U + r * W);
      uint32_t* lr = reinterpret_cast<uint32_t*>(L + r * W);
      for (int c = 2 * lane; c < W; c += 64) {
        ur[c >> 1] = (c == r ? 0u : (NEG2 & 0xffffu)) | (c + 1 == r ? 0u : (NEG2 & 0xffff0000u));  // gamma(i,i) = 0
        const bool z0 = c == r || c + 1 == r, z1 = c + 1 == r || c + 2 == r;  // L[j][j-1] = L[j][j] = 0
        lr[c >> 1] = (z0 ? 0u : (NEG2 & 0xffffu)) | (z1 ? 0u : (NEG2 & 0xffff0000u));
      }
    }
    __syncthreads();
    for (int i = tid; i < n; i += kSmallThreads) {  // prow[i] bit y: x_i may pair with base y; then x_i itself
      const int xi = xs[i];
      prow[i] = (uint8_t)(pm[xi * 4] | pm[xi * 4 + 1] << 1 | pm[xi * 4 + 2] << 2 | pm[xi * 4 + 3] << 3);
    }
    __syncthreads();
    lap(0);
    for (int d = 1; d < n; ++d) {
      // lane owns rows lane, lane + 32, ...: the cell (i, i + d) of each live row
#pragma unroll 1
      for (int i = tid; i + d < n; i += kSmallThreads) {  // (a small loop body: the loop stays in the
        const int j = i + d;                    // instruction cache)
        {
          const int xj = xs[j];                                   // issued early: the pair test needs it
          const int inner = d >= 2 ? (int)U[(i + 1) * W + j - 1] : 0;  // gamma(i+1, j-1)
          const uint4* ur = reinterpret_cast<const uint4*>(U + i * W);
          const uint4* lr = reinterpret_cast<const uint4*>(L + j * W);
          uint32_t acc0 = 0, acc1 = 0;  // gamma >= 0 and the k = i term is >= 0: 0 is neutral
#pragma unroll 1
          for (int c = i >> 3; c <= (j >> 3); ++c) {
            const uint4 a = ur[c], b = lr[c];
            acc0 = __viaddmax_s16x2(a.x, b.x, acc0);
            acc1 = __viaddmax_s16x2(a.y, b.y, acc1);
            acc0 = __viaddmax_s16x2(a.z, b.z, acc0);
            acc1 = __viaddmax_s16x2(a.w, b.w, acc1);
          }
          const uint32_t acc = __vmaxs2(acc0, acc1);
          int v = max((int)(int16_t)(acc & 0xffffu), (int)(int16_t)(acc >> 16));
          if (((prow[i] >> xj) & 1u) && d - 1 >= A.hairpin) v = max(v, inner + 1);
          U[i * W + j] = (int16_t)v;
          if (i >= 1) L[j * W + i - 1] = (int16_t)v;
        }
      }
      if (kSmallThreads == 32) __syncwarp();
      else __syncthreads();
    }
    lap(1);
    if (tid == 0) A.scores[p] = n <= 1 ? 0 : (int)U[n - 1];
    if (A.db && tid < 32) {  // canonical traceback (R-TB-NUSS), one warp, stack in shared memory
      uint8_t* db = A.db + p * A.db_stride;
      for (int k = lane; k < n; k += 32) db[k] = '.';
      int sp = 0;
      if (n > 1) {
        if (lane == 0) { stack[0] = 0; stack[1] = n - 1; }
        sp = 2;
      }
      auto gam = [&](int i, int j) -> int { return j - i < 1 ? 0 : (int)U[i * W + j]; };
      int guard = 4 * n + 8;
      while (sp > 0 && --guard > 0) {
        __syncwarp();
        const int j = stack[sp - 1], i = stack[sp - 2];
        sp -= 2;
        __syncwarp();
        if (j - i < 1) continue;
        // the four table reads of a step issued together (j - i >= 1)
        const int v = U[i * W + j], g1 = gam(i + 1, j), g2 = gam(i, j - 1), g3 = gam(i + 1, j - 1);
        const bool pr = pm[xs[i] * 4 + xs[j]] && j - i - 1 >= A.hairpin;
        int ni0 = -1, nj0 = 0, ni1 = -1, nj1 = 0;
        if (v == g1) { ni0 = i + 1; nj0 = j; }
        else if (v == g2) { ni0 = i; nj0 = j - 1; }
        else if (pr && v == g3 + 1) {
          if (lane == 0) { db[i] = '('; db[j] = ')'; }
          ni0 = i + 1; nj0 = j - 1;
        } else {
          for (int k0 = i + 1; k0 < j; k0 += 32) {  // smallest split k
            const int k = k0 + lane;
            const unsigned hit = __ballot_sync(0xffffffffu, k < j && v == (int)U[i * W + k] + (int)L[j * W + k]);
            if (hit) {
              const int kk = k0 + __ffs(hit) - 1;
              ni0 = kk + 1; nj0 = j; ni1 = i; nj1 = kk;
              break;
            }
          }
        }
        if (ni0 >= 0) {
          if (lane == 0) { stack[sp] = ni0; stack[sp + 1] = nj0; }
          sp += 2;
        }
        if (ni1 >= 0) {
          if (lane == 0) { stack[sp] = ni1; stack[sp + 1] = nj1; }
          sp += 2;
        }
      }
      if (lane == 0) A.db_len[p] = n;
    }
    lap(2);
  }
}

// One problem over the whole grid: partitions separated by grid-wide barriers
// (cooperative launch), the table in global memory (L2-resident).
__global__ void __launch_bounds__(kNussThreads) k_nuss_grid(NussArgs A, int64_t p) {
  cg::grid_group grid = cg::this_grid();
  __shared__ uint8_t pm[16];
  if (threadIdx.x < 16) pm[threadIdx.x] = A.pair_mask[threadIdx.x];
  __syncthreads();
  const uint8_t* x = A.x_cat + A.x_off[p];
  const int n = (int)(A.x_off[p + 1] - A.x_off[p]);
  int16_t* U = reinterpret_cast<int16_t*>(A.scratch);
  int16_t* L = U + (int64_t)n * (n + 1) / 2;
  const int64_t tid = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  const int64_t nthr = (int64_t)gridDim.x * blockDim.x;
  nuss_init(U, L, n, tid, nthr);
  grid.sync();
  for (int d = 1; d < n; ++d) {
    nuss_partition(U, L, x, n, d, pm, A.hairpin, tid, nthr);
    grid.sync();
  }
  if (tid == 0) A.scores[p] = n <= 1 ? 0 : (int)U[ustart(0, n) + n - 1];
  if (A.db && tid < 32) {
    int* stack = reinterpret_cast<int*>(U + table_elems(n));
    nuss_traceback_warp(U, L, x, n, pm, A.hairpin, A.db + p * A.db_stride, stack);
    if (tid == 0) A.db_len[p] = n;
  }
}

// One CTA per row: bytes of the row, then its length.
__global__ void k_copy_db(const uint8_t* db, int64_t ds, const int32_t* lens, int64_t first, int64_t count,
                          uint8_t* out, int64_t stride, int32_t* out_len) {
  for (int64_t r = blockIdx.x; r < count; r += gridDim.x) {
    const uint8_t* src = db + (first + r) * ds;
    uint8_t* dst = out + r * stride;
    const int len = lens[first + r];
    for (int k = threadIdx.x; k < len; k += blockDim.x) dst[k] = src[k];
    if (threadIdx.x == 0) out_len[r] = len;
  }
}

int num_sms(int device) {
  int v = 0;
  cudaDeviceGetAttribute(&v, cudaDevAttrMultiProcessorCount, device);
  return v > 0 ? v : 148;
}

}  // namespace

cudaError_t nuss_copy_db(const uint8_t* db, int64_t ds, const int32_t* lens, int64_t first, int64_t count,
                         uint8_t* out, int64_t stride, int32_t* out_len, cudaStream_t s, int64_t* launches) {
  if (count <= 0) return cudaSuccess;
  const int64_t grid = std::min<int64_t>(count, 148 * 16);
  ++*launches;
  k_copy_db<<<(unsigned)grid, 128, 0, s>>>(db, ds, lens, first, count, out, stride, out_len);
  return cudaGetLastError();
}

int64_t nuss_scratch_bytes(int64_t max_len, int64_t n, int device) {
  const int64_t stack_bytes = (4 * max_len + 8) * 4;
  if (max_len <= kSmemMaxN) {
    const int64_t grid = std::min<int64_t>(n, (int64_t)num_sms(device) * 4);
    return grid * stack_bytes + 256;
  }
  if (n == 1) return table_elems(max_len) * 2 + stack_bytes + 256;
  const int64_t grid = std::min<int64_t>(n, (int64_t)num_sms(device) * 2);
  return grid * (table_elems(max_len) * 2 + stack_bytes) + 256;
}

bool nuss_small_supported(int64_t max_len, int64_t n, int device) {
  return max_len <= kSmallMaxN && n <= (int64_t)num_sms(device) * 4;
}

cudaError_t nuss_small_solve(const NussArgs& A, cudaStream_t s, int64_t* launches) {
  if (A.n == 0) return cudaSuccess;
  const size_t smem = small_smem_bytes(std::max<int64_t>(A.max_len, 1));
  cudaError_t e = cudaFuncSetAttribute(k_nuss_small, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  ++*launches;
  NussArgs a2 = A;
  a2.max_len = std::max<int64_t>(A.max_len, 1);
  k_nuss_small<<<(unsigned)A.n, kSmallThreads, smem, s>>>(a2);
  return cudaGetLastError();
}

cudaError_t nuss_solve(const NussArgs& A, cudaStream_t s, int64_t* launches) {
  if (A.n == 0) return cudaSuccess;
  int dev = 0;
  cudaGetDevice(&dev);
  const int sms = num_sms(dev);
  if (A.max_len <= kSmemMaxN) {
    const size_t smem = ((A.max_len + 15) & ~15) + (size_t)table_elems(A.max_len) * 2 +
                        (A.max_len <= kSmemStackN ? (size_t)(4 * A.max_len + 8) * 4 : 0);
    cudaError_t e = cudaFuncSetAttribute(k_nuss_cta<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    const int64_t grid = std::min<int64_t>(A.n, (int64_t)sms * 4);
    // a few short problems: a small CTA keeps the per-partition barrier cheap
    const int threads = (A.n <= 2 * sms && A.max_len <= 128) ? 128 : kNussThreads;
    ++*launches;
    k_nuss_cta<true><<<(unsigned)grid, threads, smem, s>>>(A, 0);
    return cudaGetLastError();
  }
  if (A.n == 1) {
    int per_sm = 0;
    cudaError_t e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k_nuss_grid, kNussThreads, 0);
    if (e != cudaSuccess) return e;
    const int grid = sms * std::max(1, std::min(per_sm, 2));
    int64_t p = 0;
    NussArgs a2 = A;
    void* args[2] = {&a2, &p};
    ++*launches;
    return cudaLaunchCooperativeKernel((void*)k_nuss_grid, grid, kNussThreads, args, 0, s);
  }
  const size_t smem = ((A.max_len + 15) & ~15);
  const int64_t grid = std::min<int64_t>(A.n, (int64_t)sms * 2);
  ++*launches;
  k_nuss_cta<false><<<(unsigned)grid, kNussThreads, smem, s>>>(A, table_elems(A.max_len));
  return cudaGetLastError();
}

}  // namespace dpk
