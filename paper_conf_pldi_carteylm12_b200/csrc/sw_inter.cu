// Inter-task Smith–Waterman for short pairs (second half; §1.1
// L43–L47 and §6.1: "inter-task" = one problem per thread, the form CUDASW++'s hybrid
// uses for most database sequences). The paper builds intra-task kernels only and calls the
// inter-task form "algorithmically trivial"; on B200 it matters for SHORT pairs, where the
// intra-task warp kernel (k_sw16: 256 rows per warp, a 31-step ramp per strip) leaves most lanes
// idle. The plan runs it when every pair of the batch has max(|a|, |b|) <= 64 (the hybrid
// dispatch: k_sw16 above).
//
// Schedule: the anti-diagonal hyperplanes (1,1) evaluated by one thread row by row (row-major
// order is one legal linear extension of the partitions, Fig.9's scan). The row above lives in
// registers: H of NC columns (fully unrolled, static register indices), the b residues packed 4
// per word; sigma from a 32 x 32 int8 table in shared memory (one LDS per cell).
//
// Work balance (the `map` with equal work per lane): threads of a warp run in lock
// step, so a warp costs max(|a|) rows x NC columns of its 32 pairs. The pairs are visited in a
// device counting-sort order of (column bucket ceil(|b| / 8), |a|), longest first, and each warp
// runs the template for its own bucket (NC = 8 x bucket), so a warp's lanes carry pairs of one
// column bucket and nearly one row count.
//
// Columns past |b| (NC > |b|) are computed with the sentinel residue 31 (sigma = -100) and need
// no masking: by induction over row-major order, such a cell's value is below that of a cell
// visited earlier (its diagonal, upper or left neighbour minus a positive amount), so with the
// strict ">" of R-TB-SW it is never the end cell, and no valid cell reads it.
//
// Traceback retention: 2-bit codes per cell, [H != diagonal term] * 2 + [H != up term] (each a
// min(H - term, 1): no predicates, the accumulation runs on the IMAD pipe); the walk applies
// R-TB-SW's priority diagonal > up > left to them and carries H itself (H - sigma on a diagonal, H + g on a gap) and
// stops at H = 0, so "stop" needs no code. Codes: 16 B per row (NC <= 64 cells), stored
// row-major over the batch and indexed by the pair's VISITING position t ([row][t] uint4: a warp's
// 32 stores are 512 contiguous bytes; indexed by the pair id they would be scattered 16 B partial
// sectors); the sort also writes inv[p] = t for the walk. End cell: the first row-major maximum,
// kept as a per-row key max(h * 65 + 63 - j), stored at t.
#include <cstdint>
#include <cuda_runtime.h>

#include "dp_internal.h"

namespace dpk {
namespace {

constexpr int kIL = 64;                       // max(|a|, |b|) handled (columns in registers)
constexpr int kIThreads = 128;
#ifndef DP_INTER_MINB
#define DP_INTER_MINB 3
#endif
constexpr int kIMinBlocks = DP_INTER_MINB;   // CTAs per SM the register budget is sized for
constexpr int kIBuckets = kIL / 8;            // column buckets of 8
constexpr int kIKeys = kIBuckets * (kIL + 1); // sort keys: (bucket, |a|)

__device__ __forceinline__ int inter_bucket(int lb) { return lb <= 8 ? 0 : (lb - 1) >> 3; }

template <int NC, bool TB>
__device__ __forceinline__ void inter_pair(const AlignArgs& A, const int8_t* sig, int64_t p, int64_t t) {
  const uint8_t* a = A.a_cat + A.a_off[p];
  const uint8_t* b = A.b_cat + A.b_off[p];
  const int la = (int)(A.a_off[p + 1] - A.a_off[p]);
  const int lb = (int)(A.b_off[p + 1] - A.b_off[p]);
  const int g = A.gap;
  uint32_t bw[NC / 4];  // b residues, 4 per word; sentinel code 31 (sigma -100) past |b|
#pragma unroll
  for (int w = 0; w < NC / 4; ++w) {
    uint32_t v = 0;
#pragma unroll
    for (int e = 0; e < 4; ++e) {
      const int j = 4 * w + e;
      v |= (uint32_t)(j < lb ? b[j] : 31) << (8 * e);
    }
    bw[w] = v;
  }
  int H[NC];  // row i-1, then row i (columns 1..NC)
#pragma unroll
  for (int j = 0; j < NC; ++j) H[j] = 0;
  int best = 0, bi = 0, bj = 0;
  int anext = la > 0 ? a[0] : 0;  // a's residues are loaded one row ahead (the load's latency hides
                                  // behind a row of cells instead of stalling the row's first LDS)
  for (int i = 1; i <= la; ++i) {
    const int8_t* srow = sig + 32 * anext;
    if (i < la) anext = a[i];
    int hd = 0, hl = 0, rk = 0;  // H(i-1, j-1), H(i, j-1) (column 0 is 0), the row's end-cell key
    uint32_t cw[4] = {0, 0, 0, 0};
#pragma unroll
    for (int j = 0; j < NC; ++j) {
      const int s = srow[(bw[j >> 2] >> (8 * (j & 3))) & 0xff];
      const int hu = H[j];
      const int d = hd + s;
      const int m = max(hu - g, d);               // VIADDMNMX
      const int h = max(max(hl - g, m), 0);       // VIADDMNMX.RELU
      if (TB) {  // code = 2 [h != d] + [h != m]: with h != d, h == m = max(u, d) iff h == u; the walk
                 // takes diagonal > up > left
        const uint32_t nd = (uint32_t)min(h - d, 1), nu = (uint32_t)min(h - m, 1);
        cw[j >> 4] = cw[j >> 4] * 4u + (nd * 2u + nu);  // shift-accumulate: IMADs, off the ALU pipe
      }
      rk = max(rk, h * 65 + (63 - j));  // x65, not x64: an IMAD (FMA pipe) rather than a LEA (ALU)
      hd = hu;
      hl = h;
      H[j] = h;
    }
    if (rk / 65 > best) {  // strict: an earlier row keeps the tie
      best = rk / 65;
      bi = i;
      bj = 64 - rk % 65;
    }
    if (TB) {  // column 16w + r sits at bits 2 (15 - r) of word w: left-align a partial last word
      if constexpr (NC % 16 != 0) cw[NC / 16] <<= 2 * (16 - NC % 16);
    }
    if (TB) reinterpret_cast<uint4*>(A.dirs)[(int64_t)(i - 1) * A.n + t] = make_uint4(cw[0], cw[1], cw[2], cw[3]);
  }
  A.scores[p] = best;
  if (TB) reinterpret_cast<int2*>(A.ends)[t] = make_int2(bi, bj);
}

// perm: the pairs in sort order (k_inter_scatter); one pair per thread, the warp's column bucket
// (the largest of its lanes') picks the instance
template <bool TB>
__global__ void __launch_bounds__(kIThreads, kIMinBlocks) k_sw_inter(AlignArgs A, const int* perm) {
  __shared__ int8_t sig[32 * 32];
  for (int q = threadIdx.x; q < 32 * 32; q += blockDim.x) {
    const int x = q >> 5, y = q & 31;
    sig[q] = (x < A.asz && y < A.asz) ? A.sigma[x * A.asz + y] : (int8_t)-100;
  }
  __syncthreads();
  const int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  const bool live = t < A.n;
  const int64_t p = live ? perm[t] : 0;
  const int lb = live ? (int)(A.b_off[p + 1] - A.b_off[p]) : 0;
  const int bk = __reduce_max_sync(0xffffffffu, inter_bucket(lb));
  if (!live) return;
  switch (bk) {
    case 0: inter_pair<8, TB>(A, sig, p, t); break;
    case 1: inter_pair<16, TB>(A, sig, p, t); break;
    case 2: inter_pair<24, TB>(A, sig, p, t); break;
    case 3: inter_pair<32, TB>(A, sig, p, t); break;
    case 4: inter_pair<40, TB>(A, sig, p, t); break;
    case 5: inter_pair<48, TB>(A, sig, p, t); break;
    case 6: inter_pair<56, TB>(A, sig, p, t); break;
    default: inter_pair<64, TB>(A, sig, p, t); break;
  }
}

// ------------------------------------------------ the visiting order: device counting sort by key
__device__ __forceinline__ int inter_key(const AlignArgs& A, int64_t p) {
  const int la = (int)(A.a_off[p + 1] - A.a_off[p]);
  const int lb = (int)(A.b_off[p + 1] - A.b_off[p]);
  return inter_bucket(lb) * (kIL + 1) + la;
}

// Histogram and scatter privatise the 520 counters in shared memory (one global atomic per
// non-empty key and CTA): 1M pairs on ~520 keys would otherwise serialise on ~2k atomics per address.
constexpr int kISortThreads = 256, kISortItems = 8;  // pairs per CTA: 2048

__global__ void __launch_bounds__(kISortThreads) k_inter_hist(AlignArgs A, int* hist) {
  __shared__ int h[kIKeys];
  for (int k = threadIdx.x; k < kIKeys; k += blockDim.x) h[k] = 0;
  __syncthreads();
  const int64_t base = (int64_t)blockIdx.x * kISortThreads * kISortItems;
#pragma unroll
  for (int r = 0; r < kISortItems; ++r) {
    const int64_t p = base + r * kISortThreads + threadIdx.x;
    if (p < A.n) atomicAdd(&h[inter_key(A, p)], 1);
  }
  __syncthreads();
  for (int k = threadIdx.x; k < kIKeys; k += blockDim.x)
    if (h[k]) atomicAdd(&hist[k], h[k]);
}

// one CTA of 1024 threads: hist[k] <- number of pairs with a LARGER key (descending order)
__global__ void __launch_bounds__(1024) k_inter_scan(int* hist) {
  __shared__ int warp_sum[32];
  const int t = threadIdx.x, lane = t & 31, w = t >> 5;
  const int k = kIKeys - 1 - t;  // thread t holds the t-th largest key
  const int c = (k >= 0) ? hist[k] : 0;
  int x = c;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const int y = __shfl_up_sync(0xffffffffu, x, o);
    if (lane >= o) x += y;
  }
  if (lane == 31) warp_sum[w] = x;
  __syncthreads();
  if (w == 0) {
    int v = warp_sum[lane];
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const int y = __shfl_up_sync(0xffffffffu, v, o);
      if (lane >= o) v += y;
    }
    warp_sum[lane] = v;
  }
  __syncthreads();
  const int excl = x - c + (w > 0 ? warp_sum[w - 1] : 0);
  if (k >= 0) hist[k] = excl;
}

// Each CTA: local ranks from shared atomics, then one global atomic per non-empty key reserves
// the CTA's run inside that key's range (the order among equal keys is free: outputs are written
// at the pair's own index).
__global__ void __launch_bounds__(kISortThreads) k_inter_scatter(AlignArgs A, int* hist, int* perm, int* inv) {
  __shared__ int h[kIKeys];
  for (int k = threadIdx.x; k < kIKeys; k += blockDim.x) h[k] = 0;
  __syncthreads();
  const int64_t base = (int64_t)blockIdx.x * kISortThreads * kISortItems;
  int key[kISortItems], rank[kISortItems];
#pragma unroll
  for (int r = 0; r < kISortItems; ++r) {
    const int64_t p = base + r * kISortThreads + threadIdx.x;
    key[r] = p < A.n ? inter_key(A, p) : -1;
    rank[r] = key[r] >= 0 ? atomicAdd(&h[key[r]], 1) : 0;
  }
  __syncthreads();
  for (int k = threadIdx.x; k < kIKeys; k += blockDim.x)
    if (h[k]) h[k] = atomicAdd(&hist[k], h[k]);
  __syncthreads();
#pragma unroll
  for (int r = 0; r < kISortItems; ++r)
    if (key[r] >= 0) {
      const int pos = h[key[r]] + rank[r];
      const int64_t p = base + r * kISortThreads + threadIdx.x;
      perm[pos] = (int)p;
      inv[p] = pos;  // the traceback finds pair p's codes and end cell at its visiting position
    }
}

// One thread per pair: walk the codes from the end cell carrying H (ops written end -> start, then
// reversed in place). Every move leaves row i or stays in it, and the rows are visited in
// decreasing order, so the walk keeps rows i .. i-3 in registers and loads row i-4 whenever it
// moves up: four independent 16 B loads in flight instead of one dependent load per step.
__device__ __forceinline__ uint4 inter_row(const AlignArgs& A, int r, int64_t t) {
  return r >= 1 ? reinterpret_cast<const uint4*>(A.dirs)[(int64_t)(r - 1) * A.n + t] : make_uint4(0, 0, 0, 0);
}

__global__ void __launch_bounds__(kIThreads) k_sw_inter_tb(AlignArgs A, const int* inv, int64_t first, int64_t count,
                                                           uint8_t* out, int64_t stride, int32_t* out_len,
                                                           int32_t* coords) {
  const int64_t q = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (q >= count) return;
  const int64_t p = first + q;
  const uint8_t* a = A.a_cat + A.a_off[p];
  const uint8_t* b = A.b_cat + A.b_off[p];
  const int64_t t = inv[p];
  int h = A.scores[p];
  const int2 e = reinterpret_cast<const int2*>(A.ends)[t];
  int i = h > 0 ? e.x : 0, j = h > 0 ? e.y : 0;
  const int ei = i, ej = j;
  uint8_t* o = out + q * stride;
  uint4 r0 = inter_row(A, i, t), r1 = inter_row(A, i - 1, t), r2 = inter_row(A, i - 2, t),
        r3 = inter_row(A, i - 3, t);
  int n = 0;
  while (h > 0 && i > 0 && j > 0) {  // i, j > 0 whenever h > 0 (boundary H = 0); guards only
    const int wi = (j - 1) >> 4;
    const uint32_t w = wi == 0 ? r0.x : wi == 1 ? r0.y : wi == 2 ? r0.z : r0.w;
    const int c = (int)(w >> (2 * (15 - ((j - 1) & 15)))) & 3;
    if ((c & 1) && (c & 2)) {  // left: same row
      o[n++] = 'I'; h += A.gap; --j;
      continue;
    }
    if ((c & 2) == 0) {
      const int x = a[i - 1], y = b[j - 1];
      o[n++] = x == y ? 'M' : 'X';
      h -= A.sigma[x * A.asz + y];
      --j;
    } else {
      o[n++] = 'D'; h += A.gap;
    }
    --i;
    r0 = r1; r1 = r2; r2 = r3;
    r3 = inter_row(A, i - 3, t);
  }
  for (int u = 0; u < n / 2; ++u) {
    const uint8_t x = o[u];
    o[u] = o[n - 1 - u];
    o[n - 1 - u] = x;
  }
  out_len[q] = h == 0 ? n : -1 - n;  // negative: inconsistent retained state (never for a solve's own state)
  if (coords) {
    coords[4 * q] = i; coords[4 * q + 1] = j;
    coords[4 * q + 2] = ei; coords[4 * q + 3] = ej;
  }
}

}  // namespace

bool sw_inter_eligible(int64_t max_la, int64_t max_lb, int asz, int gap) {
  return max_la <= kIL && max_lb <= kIL && asz <= 31 && gap >= 1;
}

int64_t sw_inter_dir_words(int64_t max_la) { return (max_la > 0 ? max_la : 1) * 4; }

// workspace: [hist: kIKeys, padded to 4][perm: n][inv: n]
size_t sw_inter_work_bytes(int64_t n) { return (size_t)(kIKeys + 4 + 2 * n) * sizeof(int); }

cudaError_t sw_inter_solve(const AlignArgs& A, void* work, cudaStream_t s, int64_t* launches) {
  if (A.n == 0) return cudaSuccess;
  int* hist = static_cast<int*>(work);
  int* perm = hist + ((kIKeys + 3) & ~3);
  const int sort_grid = (int)((A.n + kISortThreads * kISortItems - 1) / (kISortThreads * kISortItems));
  cudaError_t e = cudaMemsetAsync(hist, 0, kIKeys * sizeof(int), s);
  if (e != cudaSuccess) return e;
  k_inter_hist<<<sort_grid, kISortThreads, 0, s>>>(A, hist);
  k_inter_scan<<<1, 1024, 0, s>>>(hist);
  k_inter_scatter<<<sort_grid, kISortThreads, 0, s>>>(A, hist, perm, perm + A.n);
  const unsigned grid = (unsigned)((A.n + kIThreads - 1) / kIThreads);
  *launches += 4;
  if (A.dirs) k_sw_inter<true><<<grid, kIThreads, 0, s>>>(A, perm);
  else k_sw_inter<false><<<grid, kIThreads, 0, s>>>(A, perm);
  return cudaGetLastError();
}

cudaError_t sw_inter_traceback(const AlignArgs& A, const void* work, int64_t first, int64_t count, uint8_t* out,
                               int64_t stride, int32_t* out_len, int32_t* coords, cudaStream_t s, int64_t* launches) {
  const int* inv = static_cast<const int*>(work) + ((kIKeys + 3) & ~3) + A.n;
  if (count == 0) return cudaSuccess;
  const int64_t grid = (count + kIThreads - 1) / kIThreads;
  ++*launches;
  k_sw_inter_tb<<<(unsigned)grid, kIThreads, 0, s>>>(A, inv, first, count, out, stride, out_len, coords);
  return cudaGetLastError();
}

}  // namespace dpk
