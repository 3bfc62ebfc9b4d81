// Pairwise alignment on the anti-diagonal schedule S(i,j) = i + j
// (§2.2, Fig.9/10 L278–L282).
//
// B200 design: one warp per problem. The schedule vector (1,1) is applied to
// TILES of R rows x 1 column: lane l owns rows [32R*strip + lR, +R) and works
// on column j at step k = j + l - 1, so every step is one hyperplane of tiles
// (A6b'), the 31 lanes above it having finished the same column one step
// earlier. The sliding window of §4.8 (w = 2 partitions) lives in registers:
// the lane keeps H of its R rows for the previous column and receives the
// boundary row from the lane above by __shfl_up_sync. Cells are max-plus:
//   SW   (§6.1): H = max(0, Hd + sigma(a_i, b_j), Hu - g, Hl - g)
//   edit (Fig.7): D = max(Dd + (a_i == b_j ? 0 : -1), Du - 1, Dl - 1),
//        d = -D (the unit-cost min-plus recursion negated; Fig.7's
//        "if s[i-1]==t[j-1] then d(i-1,j-1)" equals the min because
//        |d(i,j) - d(i-1,j)| <= 1).
// Substitution scores come from a per-problem profile P[c][i] = sigma(a_i, c)
// staged in shared memory (the substitution-matrix extension's "small table in
// shared memory", §5.1), one LDS per lane per column.
#include <cstdint>
#include <cuda_runtime.h>

#include "dp_internal.h"

namespace dpk {
namespace {

template <int R>
struct AlignSmem {
  static constexpr int kProfRows = 32 * R;
};

__device__ __forceinline__ int sext8(uint32_t w, int byte) { return (int)(int8_t)(w >> (8 * byte)); }

// Number of 32-bit direction words per lane per strip: 16/R columns per word.
__host__ __device__ constexpr int cols_per_word(int R) { return 16 / R; }

template <int R, bool LOCAL, bool TB>
__global__ void __launch_bounds__(kWarps * 32)
k_align(AlignArgs A, int n_strips_max, int smem_per_warp) {
  extern __shared__ __align__(16) uint8_t smem[];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int asz = A.asz;
  int8_t* sig_s = reinterpret_cast<int8_t*>(smem);                          // asz*asz (SW)
  const int sig_bytes = LOCAL ? ((asz * asz + 15) & ~15) : 0;
  if (LOCAL)
    for (int q = threadIdx.x; q < asz * asz; q += blockDim.x) sig_s[q] = A.sigma[q];
  __syncthreads();
  const int64_t p = (int64_t)blockIdx.x * kWarps + warp;
  if (p >= A.n) return;
  uint8_t* wbase = smem + sig_bytes + warp * smem_per_warp;
  int8_t* prof = reinterpret_cast<int8_t*>(wbase);                         // asz x 32R
  uint8_t* bseq = wbase + asz * 32 * R;                                      // max_lb
  int32_t* bnd = reinterpret_cast<int32_t*>(wbase + asz * 32 * R + ((A.max_lb + 15) & ~15));  // max_lb+1

  const uint8_t* a = A.a_cat + A.a_off[p];
  const uint8_t* b = A.b_cat + A.b_off[p];
  const int la = (int)(A.a_off[p + 1] - A.a_off[p]);
  const int lb = (int)(A.b_off[p + 1] - A.b_off[p]);
  const int g = A.gap;

  if (la == 0 || lb == 0) {
    if (lane == 0) {
      A.scores[p] = LOCAL ? 0 : (la > lb ? la : lb);
      if (TB) { A.ends[2 * p] = LOCAL ? 0 : la; A.ends[2 * p + 1] = LOCAL ? 0 : lb; }
    }
    return;
  }
  for (int q = lane; q < lb; q += 32) bseq[q] = b[q];

  const int strips = (la + 32 * R - 1) / (32 * R);
  int best = 0, bi = 0, bj = 0;  // SW: best value and first row-major argmax (TB)
  int result = 0;                // edit: D(la, lb)
  uint32_t* dirp = TB ? A.dirs + p * A.dir_stride : nullptr;
  const int wpl = (lb + cols_per_word(R) - 1) / cols_per_word(R);  // words per lane per strip

  for (int st = 0; st < strips; ++st) {
    const int row0 = st * 32 * R;          // DP rows row0+1 .. row0+32R
    const int myrow0 = row0 + lane * R;    // my DP rows myrow0+1 .. myrow0+R
    // profile P[c][r] for my rows (dead rows -> NEG)
    for (int c = 0; c < asz; ++c) {
#pragma unroll
      for (int r = 0; r < R; ++r) {
        int i = myrow0 + r;  // 0-based index into a
        int v;
        if (i < la) v = LOCAL ? sig_s[a[i] * asz + c] : (a[i] == c ? 0 : -1);
        else v = LOCAL ? -100 : -1;
        prof[c * 32 * R + lane * R + r] = (int8_t)v;
      }
    }
    __syncwarp();
    int H[R];
    int rb[R], rc[R];  // TB+SW: per-row best and its first column
#pragma unroll
    for (int r = 0; r < R; ++r) {
      H[r] = LOCAL ? 0 : -(myrow0 + r + 1);  // column 0
      if (TB && LOCAL) { rb[r] = 0; rc[r] = 0; }
    }
    int prev_up = LOCAL ? 0 : -row0;  // lane 0: H(row0, j-1) at j = 1 -> H(row0, 0)
    int last = LOCAL ? 0 : -(myrow0 + R);  // H of my last row at my current column (column 0 initially)
    uint32_t dword = 0;
    const int steps = lb + 31;
    for (int k = 0; k < steps; ++k) {
      const int j = k - lane + 1;  // my column (1-based)
      int from_above = __shfl_up_sync(0xffffffffu, last, 1);
      int up, diag;
      if (lane == 0) {
        if (st == 0) up = LOCAL ? 0 : -j;
        else up = (j >= 1 && j <= lb) ? bnd[j] : 0;
        diag = prev_up;
        prev_up = up;
      } else {
        up = from_above;
        diag = prev_up;
        prev_up = from_above;
      }
      if (j >= 1 && j <= lb) {
        const int c = bseq[j - 1];
        const int8_t* pr = prof + c * 32 * R + lane * R;
        int sig[R];
        if constexpr (R >= 4) {
#pragma unroll
          for (int w = 0; w < R / 4; ++w) {
            uint32_t word = reinterpret_cast<const uint32_t*>(pr)[w];
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
          const int left = H[r];
          const int gup = up - g, gleft = left - g;
          int h;
          if (LOCAL) h = __viaddmax_s32_relu(diag, sig[r], max(gup, gleft));
          else h = __viaddmax_s32(diag, sig[r], max(gup, gleft));
          if (TB) {
            const uint32_t code = (h == diag + sig[r]) ? 0u : (h == gup ? 1u : 2u);
            codes |= code << (2 * r);
            if (LOCAL && h > rb[r]) { rb[r] = h; rc[r] = j; }
          } else if (LOCAL) {
            best = max(best, h);
          }
          diag = left;
          H[r] = h;
          up = h;
        }
        last = up;
        if (st + 1 < strips && lane == 31) bnd[j] = up;
        if (TB) {
          const int cpw = cols_per_word(R);
          const int slot = (j - 1) % cpw;
          dword |= codes << (2 * R * slot);
          if (slot == cpw - 1 || j == lb) {
            dirp[((int64_t)st * wpl + (j - 1) / cpw) * 32 + lane] = dword;
            dword = 0;
          }
        }
      }
      __syncwarp();
    }
    if (st + 1 < strips && lane == 31) bnd[0] = LOCAL ? 0 : -(row0 + 32 * R);
    __syncwarp();
    if (TB && LOCAL) {
#pragma unroll
      for (int r = 0; r < R; ++r)
        if (rb[r] > best) { best = rb[r]; bi = myrow0 + r + 1; bj = rc[r]; }
    }
    if (!LOCAL) {
      // the lane holding DP row la in this strip keeps D(la, lb) in H
      const int rr = la - 1 - myrow0;
#pragma unroll
      for (int r = 0; r < R; ++r)
        if (rr == r) result = H[r];
    }
  }
  if (LOCAL) {
    if (TB) {
      // first maximum in row-major order: max value, then smallest i, then smallest j
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) {
        int ob = __shfl_xor_sync(0xffffffffu, best, o);
        int oi = __shfl_xor_sync(0xffffffffu, bi, o);
        int oj = __shfl_xor_sync(0xffffffffu, bj, o);
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
  } else {
    // the owner lane of row la in the last strip writes d = -D(la, lb)
    const int owner = (la - 1 - (strips - 1) * 32 * R) / R;
    if (lane == owner) {
      A.scores[p] = -result;
      if (TB) { A.ends[2 * p] = la; A.ends[2 * p + 1] = lb; }
    }
  }
}

// One thread per problem walks the stored direction codes back from the end cell.
template <int R, bool LOCAL>
__global__ void k_align_tb(AlignArgs A, int64_t first, int64_t count, uint8_t* out, int64_t stride,
                           int32_t* out_len, int32_t* coords) {
  const int64_t q = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (q >= count) return;
  const int64_t p = first + q;
  const uint8_t* a = A.a_cat + A.a_off[p];
  const uint8_t* b = A.b_cat + A.b_off[p];
  const int lb = (int)(A.b_off[p + 1] - A.b_off[p]);
  const uint32_t* dirp = A.dirs + p * A.dir_stride;
  const int ei = A.ends[2 * p], ej = A.ends[2 * p + 1];
  int i = ei, j = ej, h = A.scores[p];
  const int cpw = cols_per_word(R);
  const int wpl = (lb + cpw - 1) / cpw;
  uint8_t* o = out + q * stride;
  int64_t nops = 0;
  bool overflow = false;
  while (LOCAL ? (h > 0) : (i > 0 || j > 0)) {
    uint8_t op;
    int code;
    if (!LOCAL && i == 0) code = 2;
    else if (!LOCAL && j == 0) code = 1;
    else {
      const int row = i - 1, st = row / (32 * R), lane = (row % (32 * R)) / R, r = row % R;
      const uint32_t w = dirp[((int64_t)st * wpl + (j - 1) / cpw) * 32 + lane];
      code = (w >> (2 * R * ((j - 1) % cpw) + 2 * r)) & 3;
    }
    if (code == 0) {
      op = (a[i - 1] == b[j - 1]) ? 'M' : 'X';
      if (LOCAL) h -= A.sigma[a[i - 1] * A.asz + b[j - 1]];
      --i; --j;
    } else if (code == 1) {
      op = 'D'; h += A.gap; --i;
    } else {
      op = 'I'; h += A.gap; --j;
    }
    if (nops < stride) o[nops] = op; else overflow = true;
    ++nops;
  }
  // reverse into start -> end order
  if (!overflow)
    for (int64_t u = 0, v = nops - 1; u < v; ++u, --v) { uint8_t t = o[u]; o[u] = o[v]; o[v] = t; }
  out_len[q] = overflow ? -1 : (int32_t)nops;
  if (coords) {
    coords[4 * q] = i; coords[4 * q + 1] = j; coords[4 * q + 2] = ei; coords[4 * q + 3] = ej;
  }
}

int pick_R(int64_t max_la) {
  int64_t rows = (max_la + 31) / 32;
  if (rows <= 1) return 1;
  if (rows <= 2) return 2;
  if (rows <= 4) return 4;
  return 8;
}

int64_t align_per_warp(int R, int asz, int64_t max_la, int64_t max_lb) {
  const int64_t strips_max = (max_la + 32 * R - 1) / (32 * R);
  int64_t per_warp = (int64_t)asz * 32 * R + ((max_lb + 15) & ~int64_t(15));
  if (strips_max > 1) per_warp += (max_lb + 1) * 4;
  return (per_warp + 15) & ~int64_t(15);
}

template <int R, bool LOCAL, bool TB>
cudaError_t launch_align(const AlignArgs& A, cudaStream_t s) {
  const int strips_max = (int)((A.max_la + 32 * R - 1) / (32 * R));
  const int per_warp = (int)align_per_warp(R, A.asz, A.max_la, A.max_lb);
  const int sig_bytes = LOCAL ? ((A.asz * A.asz + 15) & ~15) : 0;
  const size_t smem = sig_bytes + (size_t)kWarps * per_warp;
  auto kern = k_align<R, LOCAL, TB>;
  cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  const int64_t blocks = (A.n + kWarps - 1) / kWarps;
  kern<<<(unsigned)blocks, kWarps * 32, smem, s>>>(A, strips_max, per_warp);
  return cudaGetLastError();
}

template <int R>
cudaError_t launch_align_r(const AlignArgs& A, cudaStream_t s) {
  const bool tb = A.dirs != nullptr;
  if (A.local) return tb ? launch_align<R, true, true>(A, s) : launch_align<R, true, false>(A, s);
  return tb ? launch_align<R, false, true>(A, s) : launch_align<R, false, false>(A, s);
}

}  // namespace

int64_t align_dir_words(int64_t max_la, int64_t max_lb) {
  const int R = pick_R(max_la);
  const int64_t strips = (max_la + 32 * R - 1) / (32 * R);
  const int64_t wpl = (max_lb + cols_per_word(R) - 1) / cols_per_word(R);
  return strips * wpl * 32;
}

size_t align_smem_bytes(int asz, bool local, int64_t max_la, int64_t max_lb) {
  const int R = pick_R(max_la);
  const size_t sig_bytes = local ? (size_t)((asz * asz + 15) & ~15) : 0;
  return sig_bytes + (size_t)kWarps * (size_t)align_per_warp(R, asz, max_la, max_lb);
}

cudaError_t align_solve(const AlignArgs& A, cudaStream_t s, int64_t* launches) {
  if (A.n == 0) return cudaSuccess;
  ++*launches;
  switch (pick_R(A.max_la)) {
    case 1: return launch_align_r<1>(A, s);
    case 2: return launch_align_r<2>(A, s);
    case 4: return launch_align_r<4>(A, s);
    default: return launch_align_r<8>(A, s);
  }
}

cudaError_t align_traceback(const AlignArgs& A, int64_t first, int64_t count, uint8_t* out, int64_t stride,
                            int32_t* out_len, int32_t* coords, cudaStream_t s, int64_t* launches) {
  if (count == 0) return cudaSuccess;
  ++*launches;
  const unsigned blocks = (unsigned)((count + 127) / 128);
  const int R = pick_R(A.max_la);
#define TBL(RR)                                                                                       \
  if (A.local) k_align_tb<RR, true><<<blocks, 128, 0, s>>>(A, first, count, out, stride, out_len, coords); \
  else k_align_tb<RR, false><<<blocks, 128, 0, s>>>(A, first, count, out, stride, out_len, coords);
  switch (R) {
    case 1: TBL(1); break;
    case 2: TBL(2); break;
    case 4: TBL(4); break;
    default: TBL(8); break;
  }
#undef TBL
  return cudaGetLastError();
}

}  // namespace dpk
