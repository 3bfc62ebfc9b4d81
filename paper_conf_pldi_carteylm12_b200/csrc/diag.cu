// The §4.7 example recurrence f(x, y) = ... f(x-1, y-1) ... (L386-L388), as the
// longest common substring (DESIGN.md R-DIAG):
//   L(i,j) = a_i == b_j ? L(i-1,j-1) + 1 : 0,   score = max L.
// Its only dependency family is (-1,-1), so both S = i (a = (1,0)) and S = j
// (a = (0,1)) are valid and each is minimal for some extents: "when nx < ny then
// Sf(x,y) = x otherwise Sf(x,y) = y" (L386-L388). The plan holds the candidates
// dp_schedule_conditional derives; the kernel evaluates the run-time condition
// per problem (L384-L386) — the candidate with the smallest box range for
// (|a|, |b|) — and sweeps that schedule's partitions: one CTA per problem
// (persistent over the batch), one partition per iteration, one barrier
// between partitions (Fig.8). Partitions of <= 4096 cells keep the window of
// one partition (§4.8: w = 1) in registers (C = 1..16 consecutive cells per
// thread); longer ones double-buffer it in shared memory as uint16.
// Choosing the schedule with fewer, longer partitions is what keeps the CTA
// busy: a 64 x 4096 pair takes 64 barriers instead of 4096.
#include <algorithm>
#include <cstdint>
#include <cuda_runtime.h>

#include "dp_internal.h"

namespace dpk {
namespace {

constexpr int kDT = 256;  // threads per CTA

__device__ __forceinline__ uint32_t prmt(uint32_t a, uint32_t b, uint32_t sel) {
  uint32_t r;
  asm("prmt.b32 %0, %1, %2, %3;" : "=r"(r) : "r"(a), "r"(b), "r"(sel));
  return r;
}

// One partition per iteration with C cells per thread in registers: thread t owns cells
// y = C t + 1 .. C t + C of every partition (nq <= 256 C). L(x, y) needs L(x-1, y-1): the
// thread's own previous values shifted by one, and for its first cell the last cell of
// thread t-1 (a shuffle; across warps through shared memory, double-buffered by parity).
// Cells past the end compare against a code no residue has and stay 0.
template <int C>
__device__ __forceinline__ int sweep_regs(const uint8_t* P, const uint8_t* Q, int np, int nq, int* xw, int tid) {
  const int lane = tid & 31, warp = tid >> 5;
  int q[C], L[C];
#pragma unroll
  for (int c = 0; c < C; ++c) {
    const int y = C * tid + c;  // 0-based column of cell c
    q[c] = y < nq ? (int)Q[y] : 0x1000;
    L[c] = 0;
  }
  int best = 0;
  for (int x = 0; x < np; ++x) {
    const int px = (int)P[x];
    int nb = __shfl_up_sync(0xffffffffu, L[C - 1], 1);
    if (lane == 0) nb = (warp > 0 && x > 0) ? xw[((x + 1) & 1) * (kDT / 32) + warp - 1] : 0;  // partition x-1's
#pragma unroll
    for (int c = C - 1; c >= 1; --c) L[c] = q[c] == px ? L[c - 1] + 1 : 0;
    L[0] = q[0] == px ? nb + 1 : 0;
#pragma unroll
    for (int c = 0; c < C; ++c) best = max(best, L[c]);
    if (lane == 31) xw[(x & 1) * (kDT / 32) + warp] = L[C - 1];
    __syncthreads();
  }
  return best;
}

// Small alphabets (asz <= 8): two cells per register (u16x2). Thread t owns cells
// 2W t .. 2W t + 2W - 1; per partition it loads, for the partition's residue px, the
// precomputed masks (0xffff in the half of a cell whose residue is px) and updates a word as
//   L' = (shift-by-one-cell(L) + 1) & mask     (PRMT, add, LOP; no carry: values < 65535)
// with a packed running max (VIMNMX.U16x2): ~2 ALU ops per cell instead of ~4.
template <int W>
__device__ __forceinline__ int sweep_packed(const uint8_t* P, const uint8_t* Q, int np, int nq, int asz,
                                            uint32_t* msk, uint32_t* xw, int tid) {
  const int lane = tid & 31, warp = tid >> 5;
  // masks [code][w][tid] (conflict-free: consecutive threads, consecutive words)
  for (int code = 0; code < asz; ++code)
#pragma unroll
    for (int w = 0; w < W; ++w) {
      const int y0 = 2 * W * tid + 2 * w;
      const uint32_t lo = (y0 < nq && Q[y0] == code) ? 0xffffu : 0u;
      const uint32_t hi = (y0 + 1 < nq && Q[y0 + 1] == code) ? 0xffff0000u : 0u;
      msk[(code * W + w) * kDT + tid] = lo | hi;
    }
  __syncthreads();
  uint32_t L[W], acc = 0;
#pragma unroll
  for (int w = 0; w < W; ++w) L[w] = 0;
  for (int x = 0; x < np; ++x) {
    const int px = (int)P[x];
    uint32_t m[W];
#pragma unroll
    for (int w = 0; w < W; ++w) m[w] = px < asz ? msk[(px * W + w) * kDT + tid] : 0u;
    uint32_t nb = __shfl_up_sync(0xffffffffu, L[W - 1], 1);
    if (lane == 0) nb = (warp > 0 && x > 0) ? xw[((x + 1) & 1) * (kDT / 32) + warp - 1] : 0u;  // partition x-1's
#pragma unroll
    for (int w = W - 1; w >= 1; --w) L[w] = (prmt(L[w - 1], L[w], 0x5432u) + 0x00010001u) & m[w];
    L[0] = (prmt(nb, L[0], 0x5432u) + 0x00010001u) & m[0];
#pragma unroll
    for (int w = 0; w < W; ++w) acc = __vmaxu2(acc, L[w]);
    if (lane == 31) xw[(x & 1) * (kDT / 32) + warp] = L[W - 1];
    __syncthreads();
  }
  return (int)max(acc & 0xffffu, acc >> 16);
}

__global__ void __launch_bounds__(kDT) k_diag(DiagArgs A) {
  extern __shared__ __align__(16) uint8_t dsm[];
  const int64_t cap = A.max_len;
  uint16_t* row0 = reinterpret_cast<uint16_t*>(dsm);
  uint16_t* row1 = row0 + cap + 8;
  const size_t region = max((size_t)(2 * (cap + 8) * 2), (A.asz >= 1 && A.asz <= 8) ? (size_t)A.asz * 8 * kDT * 4 : 0);
  uint8_t* qs = dsm + region;
  uint8_t* ps = qs + ((cap + 15) & ~int64_t(15));
  __shared__ int red[kDT / 32];
  __shared__ uint32_t xw[2 * (kDT / 32)];
  const int tid = threadIdx.x;
  for (int64_t p = blockIdx.x; p < A.n; p += gridDim.x) {
    const int64_t la = A.a_off[p + 1] - A.a_off[p], lb = A.b_off[p + 1] - A.b_off[p];
    // run-time schedule choice (§4.7): the candidate with the smallest box range sum |a_i| (n_i - 1)
    int k = 0;
    if (A.force >= 0 && A.force < A.ncand) {
      k = A.force;
    } else {
      int64_t bg = INT64_MAX;
      for (int c = 0; c < A.ncand; ++c) {
        const int64_t g = (int64_t)abs(A.cand[c][0]) * (la > 0 ? la - 1 : 0) + (int64_t)abs(A.cand[c][1]) * (lb > 0 ? lb - 1 : 0);
        if (g < bg) { bg = g; k = c; }
      }
    }
    // S = i: the partitions are the rows i = 1..|a| (cells along j); S = j: the columns.
    // L is symmetric in (a, b), so the column sweep is the row sweep of the swapped pair.
    const bool by_row = A.cand[k][0] != 0;
    const uint8_t* P = by_row ? A.a_cat + A.a_off[p] : A.b_cat + A.b_off[p];
    const uint8_t* Q = by_row ? A.b_cat + A.b_off[p] : A.a_cat + A.a_off[p];
    const int np = (int)(by_row ? la : lb), nq = (int)(by_row ? lb : la);
    __syncthreads();  // the previous problem's buffers are free
    for (int y = tid; y < nq; y += kDT) qs[y] = Q[y];
    for (int y = tid; y < np; y += kDT) ps[y] = P[y];
    const bool packed = A.asz >= 1 && A.asz <= 8 && nq <= 16 * kDT;
    const bool regs = nq <= 16 * kDT;
    if (!regs)
      for (int y = tid; y <= nq; y += kDT) { row0[y] = 0; row1[y] = 0; }
    __syncthreads();
    int best = 0;
    if (packed) {
      uint32_t* msk = reinterpret_cast<uint32_t*>(row0);  // the window rows are free on this path
      if (nq <= 2 * kDT) best = sweep_packed<1>(ps, qs, np, nq, A.asz, msk, xw, tid);
      else if (nq <= 4 * kDT) best = sweep_packed<2>(ps, qs, np, nq, A.asz, msk, xw, tid);
      else if (nq <= 8 * kDT) best = sweep_packed<4>(ps, qs, np, nq, A.asz, msk, xw, tid);
      else best = sweep_packed<8>(ps, qs, np, nq, A.asz, msk, xw, tid);
    } else if (regs) {
      if (nq <= kDT) best = sweep_regs<1>(ps, qs, np, nq, reinterpret_cast<int*>(xw), tid);
      else if (nq <= 2 * kDT) best = sweep_regs<2>(ps, qs, np, nq, reinterpret_cast<int*>(xw), tid);
      else if (nq <= 4 * kDT) best = sweep_regs<4>(ps, qs, np, nq, reinterpret_cast<int*>(xw), tid);
      else if (nq <= 8 * kDT) best = sweep_regs<8>(ps, qs, np, nq, reinterpret_cast<int*>(xw), tid);
      else best = sweep_regs<16>(ps, qs, np, nq, reinterpret_cast<int*>(xw), tid);
    } else {
      // long partitions: the window row in shared memory, every thread on a strided slice
      uint16_t* prev = row0;
      uint16_t* cur = row1;
      for (int x = 1; x <= np; ++x) {  // partition x: every cell (x, y) at once, then a barrier
        const uint8_t px = ps[x - 1];
        for (int y = tid + 1; y <= nq; y += kDT) {
          const int v = qs[y - 1] == px ? prev[y - 1] + 1 : 0;
          cur[y] = (uint16_t)v;
          best = max(best, v);
        }
        __syncthreads();
        uint16_t* t = prev; prev = cur; cur = t;
      }
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) best = max(best, __shfl_xor_sync(0xffffffffu, best, o));
    if ((tid & 31) == 0) red[tid >> 5] = best;
    __syncthreads();
    if (tid == 0) {
      int b = 0;
      for (int w = 0; w < kDT / 32; ++w) b = max(b, red[w]);
      A.scores[p] = b;
    }
  }
}

}  // namespace

size_t diag_smem_bytes(int64_t max_len, int asz) {
  // window rows (generic path) or, aliased, the masks of the packed path (asz x 8 words x 256)
  const size_t rows = (size_t)(2 * (max_len + 8) * 2);
  const size_t masks = (asz >= 1 && asz <= 8) ? (size_t)asz * 8 * kDT * 4 : 0;
  return std::max(rows, masks) + 2 * ((max_len + 15) & ~int64_t(15));
}

cudaError_t diag_solve(const DiagArgs& A, cudaStream_t s, int64_t* launches) {
  if (A.n == 0) return cudaSuccess;
  const size_t smem = diag_smem_bytes(A.max_len, A.asz);
  cudaError_t e = cudaFuncSetAttribute(k_diag, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  int dev = 0, sms = 0, per_sm = 0;
  if ((e = cudaGetDevice(&dev)) != cudaSuccess) return e;
  if ((e = cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev)) != cudaSuccess) return e;
  if ((e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k_diag, kDT, smem)) != cudaSuccess) return e;
  if (per_sm < 1) return cudaErrorInvalidConfiguration;
  const int64_t grid = A.n < (int64_t)per_sm * sms ? A.n : (int64_t)per_sm * sms;
  ++*launches;
  k_diag<<<(unsigned)grid, kDT, smem, s>>>(A);
  return cudaGetLastError();
}

}  // namespace dpk
