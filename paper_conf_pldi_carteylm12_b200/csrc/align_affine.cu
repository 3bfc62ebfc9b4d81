// Smith–Waterman with affine gaps (Gotoh; SURVEY.md §8(f) NEXT rank 1,
// DESIGN.md R-SW-AFFINE): three mutually recursive tables
//   E(i,j) = max(E(i,j-1) - ge, H(i,j-1) - go - ge)
//   F(i,j) = max(F(i-1,j) - ge, H(i-1,j) - go - ge)
//   H(i,j) = max(0, H(i-1,j-1) + sigma(a_i, b_j), E(i,j), F(i,j))
// The cross-cell dependence offsets of all three tables are (0,-1), (-1,0),
// (-1,-1) — the linear recursion's families — so the front end derives the
// same schedule (1,1); the same-cell references H <- E, F fix the evaluation
// order inside a cell (E and F before H). Layout as k_align: one warp per
// problem, lane l owns rows [32R strip + lR, +R) and works on column j at step
// j + l - 1; H and F of the lane's last row travel down the warp by
// __shfl_up_sync, E stays with its row. int32 throughout.
// Traceback retention: 4 bits per cell (H source: diagonal / F / E; F opened
// here; E opened here), walked by one thread per problem (k_align_affine_tb).
#include <cstdint>
#include <cuda_runtime.h>

#include "dp_internal.h"

namespace dpk {
namespace {

constexpr int kNegInf = -(1 << 28);  // E(i,0), F(0,j)

__device__ __forceinline__ int sext8(uint32_t w, int byte) { return (int)(int8_t)(w >> (8 * byte)); }
__host__ __device__ constexpr int acols_per_word(int R) { return 8 / R; }  // 4 bits x R rows per column

template <int R, bool TB>
__global__ void __launch_bounds__(kWarps * 32) k_align_affine(AlignArgs A, int smem_per_warp) {
  extern __shared__ __align__(16) uint8_t smem[];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int asz = A.asz;
  int8_t* sig_s = reinterpret_cast<int8_t*>(smem);
  const int sig_bytes = (asz * asz + 15) & ~15;
  for (int q = threadIdx.x; q < asz * asz; q += blockDim.x) sig_s[q] = A.sigma[q];
  __syncthreads();
  const int64_t p = (int64_t)blockIdx.x * kWarps + warp;
  if (p >= A.n) return;
  uint8_t* wbase = smem + sig_bytes + warp * smem_per_warp;
  int8_t* prof = reinterpret_cast<int8_t*>(wbase);                          // asz x 32R
  uint8_t* bseq = wbase + asz * 32 * R;                                       // max_lb
  int32_t* bnd = reinterpret_cast<int32_t*>(wbase + asz * 32 * R + ((A.max_lb + 15) & ~15));  // H, F of row 32R st
  const uint8_t* a = A.a_cat + A.a_off[p];
  const uint8_t* b = A.b_cat + A.b_off[p];
  const int la = (int)(A.a_off[p + 1] - A.a_off[p]);
  const int lb = (int)(A.b_off[p + 1] - A.b_off[p]);
  const int ge = A.gap_ext, goe = A.gap_open + A.gap_ext;
  if (la == 0 || lb == 0) {
    if (lane == 0) {
      A.scores[p] = 0;
      if (TB) { A.ends[2 * p] = 0; A.ends[2 * p + 1] = 0; }
    }
    return;
  }
  for (int q = lane; q < lb; q += 32) bseq[q] = b[q];
  const int strips = (la + 32 * R - 1) / (32 * R);
  int best = 0, bi = 0, bj = 0;
  uint32_t* dirp = TB ? A.dirs + p * A.dir_stride : nullptr;
  const int cpw = acols_per_word(R);
  const int wpl = (lb + cpw - 1) / cpw;
  for (int st = 0; st < strips; ++st) {
    const int row0 = st * 32 * R;
    const int myrow0 = row0 + lane * R;
    for (int c = 0; c < asz; ++c) {
#pragma unroll
      for (int r = 0; r < R; ++r) {
        const int i = myrow0 + r;
        prof[c * 32 * R + lane * R + r] = (int8_t)(i < la ? sig_s[a[i] * asz + c] : -100);
      }
    }
    __syncwarp();
    int H[R], E[R], rb[R], rc[R];
#pragma unroll
    for (int r = 0; r < R; ++r) { H[r] = 0; E[r] = kNegInf; rb[r] = 0; rc[r] = 0; }
    int prev_up = 0;             // H(row above, j - 1)
    int lastH = 0, lastF = kNegInf;  // H, F of my last row at my current column
    uint32_t dword = 0;
    for (int k = 0; k < lb + 31; ++k) {
      const int j = k - lane + 1;
      const int fH = __shfl_up_sync(0xffffffffu, lastH, 1);
      const int fF = __shfl_up_sync(0xffffffffu, lastF, 1);
      int hup, fup, diag;
      if (lane == 0) {
        const bool in = j >= 1 && j <= lb;
        hup = (st == 0 || !in) ? 0 : bnd[2 * j];
        fup = (st == 0 || !in) ? kNegInf : bnd[2 * j + 1];
        diag = prev_up;
        prev_up = hup;
      } else {
        hup = fH; fup = fF;
        diag = prev_up;
        prev_up = fH;
      }
      if (j >= 1 && j <= lb) {
        const int c = bseq[j - 1];
        const int8_t* pr = prof + c * 32 * R + lane * R;
        int sig[R];
        if constexpr (R >= 4) {
#pragma unroll
          for (int w = 0; w < R / 4; ++w) {
            const uint32_t word = reinterpret_cast<const uint32_t*>(pr)[w];
#pragma unroll
            for (int q = 0; q < 4; ++q) sig[4 * w + q] = sext8(word, q);
          }
        } else {
#pragma unroll
          for (int r = 0; r < R; ++r) sig[r] = pr[r];
        }
        uint32_t codes = 0;
#pragma unroll
        for (int r = 0; r < R; ++r) {
          const int eo = H[r] - goe, fo = hup - goe;
          const int e = max(E[r] - ge, eo);
          const int f = max(fup - ge, fo);
          const int h = __viaddmax_s32_relu(diag, sig[r], max(e, f));
          if (TB) {
            const uint32_t src = (h == diag + sig[r]) ? 0u : (h == f ? 1u : 2u);
            codes |= (src | ((f == fo) ? 4u : 0u) | ((e == eo) ? 8u : 0u)) << (4 * r);
            if (h > rb[r]) { rb[r] = h; rc[r] = j; }
          } else {
            best = max(best, h);
          }
          diag = H[r];
          H[r] = h;
          E[r] = e;
          hup = h;
          fup = f;
        }
        lastH = hup;
        lastF = fup;
        if (st + 1 < strips && lane == 31) { bnd[2 * j] = hup; bnd[2 * j + 1] = fup; }
        if (TB) {
          const int slot = (j - 1) % cpw;
          dword |= codes << (4 * R * slot);
          if (slot == cpw - 1 || j == lb) {
            dirp[((int64_t)st * wpl + (j - 1) / cpw) * 32 + lane] = dword;
            dword = 0;
          }
        }
      }
      __syncwarp();
    }
    __syncwarp();
    if (TB) {
#pragma unroll
      for (int r = 0; r < R; ++r)
        if (rb[r] > best) { best = rb[r]; bi = myrow0 + r + 1; bj = rc[r]; }
    }
  }
  if (TB) {
    // first maximum in row-major order: max value, then smallest i, then smallest j
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
      const int ob = __shfl_xor_sync(0xffffffffu, best, o);
      const int oi = __shfl_xor_sync(0xffffffffu, bi, o);
      const int oj = __shfl_xor_sync(0xffffffffu, bj, o);
      if (ob > best || (ob == best && (oi < bi || (oi == bi && oj < bj)))) { best = ob; bi = oi; bj = oj; }
    }
    if (lane == 0) {
      A.scores[p] = best;
      A.ends[2 * p] = best > 0 ? bi : 0;
      A.ends[2 * p + 1] = best > 0 ? bj : 0;
    }
  } else {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) best = max(best, __shfl_xor_sync(0xffffffffu, best, o));
    if (lane == 0) A.scores[p] = best;
  }
}

// One thread per problem walks the three-state machine back from the end cell
// (DESIGN.md R-TB-SWA); h (in H) or f / e (in a gap state) are tracked exactly.
template <int R>
__global__ void k_align_affine_tb(AlignArgs A, int64_t first, int64_t count, uint8_t* out, int64_t stride,
                                  int32_t* out_len, int32_t* coords) {
  const int64_t q = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (q >= count) return;
  const int64_t p = first + q;
  const uint8_t* a = A.a_cat + A.a_off[p];
  const uint8_t* b = A.b_cat + A.b_off[p];
  const int lb = (int)(A.b_off[p + 1] - A.b_off[p]);
  const uint32_t* dirp = A.dirs + p * A.dir_stride;
  const int ei = A.ends[2 * p], ej = A.ends[2 * p + 1];
  const int ge = A.gap_ext, goe = A.gap_open + A.gap_ext;
  const int cpw = acols_per_word(R);
  const int wpl = (lb + cpw - 1) / cpw;
  auto code_at = [&](int i, int j) -> uint32_t {
    const int row = i - 1, st = row / (32 * R), lane = (row % (32 * R)) / R, r = row % R;
    const uint32_t w = dirp[((int64_t)st * wpl + (j - 1) / cpw) * 32 + lane];
    return (w >> (4 * R * ((j - 1) % cpw) + 4 * r)) & 15u;
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
      if (src == 0) {
        op = (a[i - 1] == b[j - 1]) ? 'M' : 'X';
        v -= A.sigma[a[i - 1] * A.asz + b[j - 1]];
        --i; --j;
      } else {
        state = src == 1 ? 1 : 2;  // H(i,j) == F(i,j) or E(i,j): same value, no move
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

int pick_R_affine(int64_t max_la) {
  const int64_t rows = (max_la + 31) / 32;
  if (rows <= 1) return 1;
  if (rows <= 2) return 2;
  if (rows <= 4) return 4;
  return 8;
}

int64_t affine_per_warp(int R, int asz, int64_t max_la, int64_t max_lb) {
  const int64_t strips_max = (max_la + 32 * R - 1) / (32 * R);
  int64_t per_warp = (int64_t)asz * 32 * R + ((max_lb + 15) & ~int64_t(15));
  if (strips_max > 1) per_warp += (max_lb + 1) * 8;
  return (per_warp + 15) & ~int64_t(15);
}

template <int R, bool TB>
cudaError_t launch_affine(const AlignArgs& A, cudaStream_t s) {
  const int per_warp = (int)affine_per_warp(R, A.asz, A.max_la, A.max_lb);
  const size_t smem = ((A.asz * A.asz + 15) & ~15) + (size_t)kWarps * per_warp;
  auto kern = k_align_affine<R, TB>;
  cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  kern<<<(unsigned)((A.n + kWarps - 1) / kWarps), kWarps * 32, smem, s>>>(A, per_warp);
  return cudaGetLastError();
}

}  // namespace

int64_t align_affine_dir_words(int64_t max_la, int64_t max_lb) {
  const int R = pick_R_affine(max_la);
  const int64_t strips = (max_la + 32 * R - 1) / (32 * R);
  const int64_t wpl = (max_lb + acols_per_word(R) - 1) / acols_per_word(R);
  return strips * wpl * 32;
}

size_t align_affine_smem_bytes(int asz, int64_t max_la, int64_t max_lb) {
  return (size_t)((asz * asz + 15) & ~15) + (size_t)kWarps * (size_t)affine_per_warp(pick_R_affine(max_la), asz, max_la, max_lb);
}

cudaError_t align_affine_solve(const AlignArgs& A, cudaStream_t s, int64_t* launches) {
  if (A.n == 0) return cudaSuccess;
  ++*launches;
  const bool tb = A.dirs != nullptr;
  switch (pick_R_affine(A.max_la)) {
    case 1: return tb ? launch_affine<1, true>(A, s) : launch_affine<1, false>(A, s);
    case 2: return tb ? launch_affine<2, true>(A, s) : launch_affine<2, false>(A, s);
    case 4: return tb ? launch_affine<4, true>(A, s) : launch_affine<4, false>(A, s);
    default: return tb ? launch_affine<8, true>(A, s) : launch_affine<8, false>(A, s);
  }
}

cudaError_t align_affine_traceback(const AlignArgs& A, int64_t first, int64_t count, uint8_t* out, int64_t stride,
                                   int32_t* out_len, int32_t* coords, cudaStream_t s, int64_t* launches) {
  if (count == 0) return cudaSuccess;
  ++*launches;
  const unsigned blocks = (unsigned)((count + 127) / 128);
  switch (pick_R_affine(A.max_la)) {
    case 1: k_align_affine_tb<1><<<blocks, 128, 0, s>>>(A, first, count, out, stride, out_len, coords); break;
    case 2: k_align_affine_tb<2><<<blocks, 128, 0, s>>>(A, first, count, out, stride, out_len, coords); break;
    case 4: k_align_affine_tb<4><<<blocks, 128, 0, s>>>(A, first, count, out, stride, out_len, coords); break;
    default: k_align_affine_tb<8><<<blocks, 128, 0, s>>>(A, first, count, out, stride, out_len, coords); break;
  }
  return cudaGetLastError();
}

}  // namespace dpk
