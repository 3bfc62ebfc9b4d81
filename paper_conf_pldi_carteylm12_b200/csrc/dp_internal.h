// Internal launcher interface between the C-ABI layer (api.cu) and the
// kernels (align.cu, nussinov.cu, hmm.cu). Not installed; not part of dp.h.
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

namespace dpk {

// Diagnostic phase clock (DP_*_TIMING): per-phase SM cycles of lane 0 of every warp,
// summed into 8 device counters at the end of the kernel. Off (dbg == nullptr) it costs
// one predicated branch per lap.
struct PhaseClock {
  unsigned long long* dbg;
  long long t;
  __device__ __forceinline__ void start() { if (dbg) t = clock64(); }
  // off (dbg == nullptr) only the pointer stays live; on, lane 0 of every warp adds its lap
  __device__ __forceinline__ void lap(int q) {
    if (dbg) {
      const long long u = clock64();
      if ((threadIdx.x & 31) == 0) atomicAdd(dbg + q, (unsigned long long)(u - t));
      t = u;
    }
  }
  __device__ __forceinline__ void count(int q) { if (dbg && (threadIdx.x & 31) == 0) atomicAdd(dbg + q, 1ull); }
  __device__ __forceinline__ void flush(int) {}
};

constexpr int kWarps = 8;  // warps per CTA for the warp-per-problem kernels

// ---------------------------------------------------------------- alignment
struct AlignArgs {
  int64_t n;
  const uint8_t *a_cat, *b_cat;
  const int64_t *a_off, *b_off;
  int64_t max_la, max_lb;
  const int8_t* sigma;   // device [asz x asz] (SW) or nullptr (edit)
  int asz;
  int gap;
  bool local;            // SW (true) vs edit distance (false)
  int gap_open, gap_ext; // affine SW (align_affine.cu)
  int32_t* scores;
  // traceback retention (nullptr when not wanted)
  uint32_t* dirs;        // direction codes, 2 bits per cell
  int64_t dir_stride;    // words per problem
  int32_t* ends;         // n x 2 (end_i, end_j)
};
int64_t align_dir_words(int64_t max_la, int64_t max_lb);  // words per problem for `dirs`
size_t align_smem_bytes(int asz, bool local, int64_t max_la, int64_t max_lb);  // k_align dynamic smem per CTA
size_t align_affine_smem_bytes(int asz, int64_t max_la, int64_t max_lb);        // k_align_affine
int64_t align_affine_dir_words(int64_t max_la, int64_t max_lb);  // affine: 4 bits per cell
cudaError_t align_affine_solve(const AlignArgs& a, cudaStream_t s, int64_t* launches);
cudaError_t align_affine_traceback(const AlignArgs& a, int64_t first, int64_t count, uint8_t* out, int64_t stride,
                                   int32_t* out_len, int32_t* coords, cudaStream_t s, int64_t* launches);
// packed s16x2 affine SW (affine16.cu): two problems per warp, keyed codes; dirs strided per GROUP
bool affine16_eligible(int64_t max_la, int64_t max_lb, const int8_t* sigma_host, int asz, int go, int ge);
size_t affine16_smem_bytes(int asz, int64_t max_la, int64_t max_lb);
int64_t affine16_dir_words(int64_t max_la, int64_t max_lb);  // words per group of two problems
cudaError_t affine16_solve(const AlignArgs& a, cudaStream_t s, int64_t* launches);
cudaError_t affine16_traceback(const AlignArgs& a, int64_t first, int64_t count, uint8_t* out, int64_t stride,
                               int32_t* out_len, int32_t* coords, cudaStream_t s, int64_t* launches);
cudaError_t align_solve(const AlignArgs& a, cudaStream_t s, int64_t* launches);
cudaError_t align_traceback(const AlignArgs& a, int64_t first, int64_t count, uint8_t* out, int64_t stride,
                            int32_t* out_len, int32_t* coords, cudaStream_t s, int64_t* launches);

// ---------------------------------------------------------------- inter-task SW (sw_inter.cu): one pair per thread
bool sw_inter_eligible(int64_t max_la, int64_t max_lb, int asz, int gap);  // max(|a|, |b|) <= 64, gap >= 1
int64_t sw_inter_dir_words(int64_t max_la);                                  // code words per problem (16 B per row)
size_t sw_inter_work_bytes(int64_t n);                                       // sort workspace (histogram + order)
cudaError_t sw_inter_solve(const AlignArgs& a, void* work, cudaStream_t s, int64_t* launches);
cudaError_t sw_inter_traceback(const AlignArgs& a, const void* work, int64_t first, int64_t count, uint8_t* out,
                               int64_t stride,
                               int32_t* out_len, int32_t* coords, cudaStream_t s, int64_t* launches);

// ---------------------------------------------------------------- packed SW (two problems per warp)
struct Sw16Args {
  int64_t n;
  const uint8_t *a_cat, *b_cat;
  const int64_t *a_off, *b_off;
  int64_t max_la, max_lb;
  const int8_t* sigma;   // device [asz x asz]
  int asz, gap;
  int smem_per_warp;
  int32_t* scores;
  // traceback checkpoints (nullptr in score-only mode)
  uint32_t* rowck;       // [groups][strips][8 bands][max_lb]    G of each 32-row band's bottom row (packed pair)
  uint32_t* colck;       // [groups][strips][nslab][256]         G at each lane's checkpoint column 32 s - lane
  uint32_t* slabbest;    // [groups][strips][nslab][32]           per-lane best G per slab (32 sweep steps)
  uint32_t* corner;      // [groups][strips][nslab][32]           G of the row above the lane at its checkpoint column
  uint32_t* lanebest;    // [groups][strips][32]                  per-lane best G over the strip
  int64_t strips_max, nslab_max;
  unsigned long long* tb_ctr;  // traceback work queues (two 64-bit counters, zeroed per launch)
  unsigned long long* dbg = nullptr;  // DP_SW_TIMING: traceback phase cycles (8 counters), else nullptr
};
bool sw16_eligible(int64_t max_la, int64_t max_lb, const int8_t* sigma_host, int asz, int gap, bool want_tb);
int sw16_smem_per_warp(int asz, int64_t max_la, int64_t max_lb);
size_t sw16_smem_bytes(int asz, int64_t max_la, int64_t max_lb);  // k_sw16 dynamic smem per CTA
void sw16_state_words(int64_t n, int64_t max_la, int64_t max_lb, int64_t* strips, int64_t* nslab, int64_t* rowck,
                      int64_t* colck, int64_t* slabbest);
cudaError_t sw16_solve(const Sw16Args& a, bool tb, cudaStream_t s, int64_t* launches);
cudaError_t sw16_traceback(const Sw16Args& a, int64_t first, int64_t count, uint8_t* out, int64_t stride,
                           int32_t* out_len, int32_t* coords, cudaStream_t s, int64_t* launches);

// ---------------------------------------------------------------- diagonal-only (§4.7)
struct DiagArgs {
  int64_t n;
  const uint8_t *a_cat, *b_cat;
  const int64_t *a_off, *b_off;
  int64_t max_len;       // max over the batch of max(|a|, |b|)
  int32_t* scores;
  int32_t cand[24][2];   // §4.7 candidate schedules (dp_schedule_conditional)
  int ncand;
  int force;             // -1: run-time choice per problem; else that candidate (diagnostic)
  int asz;               // alphabet size if known (<= 8: packed two-cells-per-register path), else 0
};
size_t diag_smem_bytes(int64_t max_len, int asz);
cudaError_t diag_solve(const DiagArgs& a, cudaStream_t s, int64_t* launches);

// ---------------------------------------------------------------- Nussinov
struct NussArgs {
  int64_t n;
  const uint8_t* x_cat;
  const int64_t* x_off;
  int64_t max_len;
  const uint8_t* pair_mask;  // device [16]
  int hairpin;
  int32_t* scores;
  uint8_t* db;               // dot-brackets (n x db_stride) or nullptr
  int64_t db_stride;
  int32_t* db_len;
  void* scratch;             // global table scratch for large n
  int64_t scratch_bytes;
  unsigned long long* round_ns;  // optional: %globaltimer at each tile-diagonal round (grid sweep)
  unsigned long long* dbg = nullptr;  // DP_NUSS_TIMING: batch-kernel phase cycles (8 counters)
  int tbw = 0;                        // grid traceback window (8/16/32; DP_NUSS_TBW), 0 = default
  int* queue = nullptr;               // batch work queue counter (set by the launcher)
  const int* perm = nullptr;          // problems in decreasing length (set by the launcher)
};
int64_t nuss_scratch_bytes(int64_t max_len, int64_t n, int device);
bool nuss_tiled_supported(int64_t max_len);
int64_t nuss_tiled_scratch_bytes(int64_t max_len, int64_t n, int device);
cudaError_t nuss_tiled_solve(const NussArgs& a, cudaStream_t s, int64_t* launches);
// a few mid-length problems, one thread-block cluster each, tables in distributed shared memory
bool nuss_cluster_supported(int64_t max_len, int64_t n, int device);
int64_t nuss_cluster_scratch_bytes(int64_t max_len, int64_t n);
cudaError_t nuss_cluster_solve(const NussArgs& a, cudaStream_t s, int64_t* launches);
cudaError_t nuss_solve(const NussArgs& a, cudaStream_t s, int64_t* launches);
// one CTA per problem, table + traceback in shared memory (latency regime: max_len <= 128, few problems)
bool nuss_small_supported(int64_t max_len, int64_t n, int device);
cudaError_t nuss_small_solve(const NussArgs& a, cudaStream_t s, int64_t* launches);
// copy rows [first, first+count) of the dot-bracket scratch (row stride ds) and their lengths
cudaError_t nuss_copy_db(const uint8_t* db, int64_t ds, const int32_t* lens, int64_t first, int64_t count,
                         uint8_t* out, int64_t stride, int32_t* out_len, cudaStream_t s, int64_t* launches);

// ---------------------------------------------------------------- HMM
struct HmmArgs {
  int64_t n;
  const uint8_t* x_cat;
  const int64_t* x_off;
  int64_t max_len;
  int S, K;
  const float *pi, *A, *E;          // device, forward
  const int32_t *lpi, *lA, *lE;     // device, Viterbi
  float* ll_out;                    // forward
  int32_t* vit_out;                 // Viterbi
  uint8_t* bp;                      // Viterbi back-pointers (n x max_len x 64) or nullptr
  int32_t* final_state;             // n
  uint8_t* path = nullptr;          // Viterbi: the walked state path (n x max_len), written by k_viterbi
  unsigned long long* dbg = nullptr;  // diagnostic step timestamps (DP_HMM_TIMING), else nullptr
  int ns_override = 0;                // diagnostic: sequences per warp of the SIMT kernels (DP_HMM_NS)
  int tc_smem_kb = -1;                // shared memory the tcgen05 forward reserves per CTA (-1: default)
  // Viterbi in s16x2 (hmm_vit16.cu): clamp C (> 0: the 16-bit kernel runs), saturating emission add,
  // and its per-position rows for the walk ((n+1)/2 pairs x max_len x 64 packed words) or nullptr
  int v16_C = 0;
  int v16_sat = 0;
  uint32_t* rows16 = nullptr;
};
cudaError_t hmm_forward(const HmmArgs& a, cudaStream_t s, int64_t* launches);
bool hmm_forward_tc_supported(int S);
cudaError_t hmm_forward_tc(const HmmArgs& a, cudaStream_t s, int64_t* launches);  // tcgen05 path
cudaError_t hmm_viterbi(const HmmArgs& a, cudaStream_t s, int64_t* launches);
int vit16_clamp(const int32_t* lA, const int32_t* lE, int S, int K, int* sat);  // host: C, or 0 if not exact
cudaError_t hmm_viterbi16(const HmmArgs& a, cudaStream_t s, int64_t* launches);
cudaError_t hmm_viterbi_traceback(const HmmArgs& a, int64_t first, int64_t count, uint8_t* out, int64_t stride,
                                  int32_t* out_len, cudaStream_t s, int64_t* launches);

// ---------------------------------------------------------------- profile HMM (phmm.cu)
struct PhmmArgs {
  int64_t n;
  const uint8_t* x_cat;
  const int64_t* x_off;
  int64_t max_len;
  int L, K;
  const float* trans;    // device [(L+1) x 9]: from (M_j, I_j, D_j) to (M_{j+1}, I_j, D_{j+1})
  const float* emit_m;   // device [(L+1) x K] (row 0 unused)
  const float* emit_i;   // device [(L+1) x K]
  float* ll_out;         // n natural-log likelihoods
  int rows_tab;          // set by the launcher
};
size_t phmm_smem_bytes(int L, int K, int64_t max_len);
cudaError_t phmm_forward(const PhmmArgs& a, cudaStream_t s, int64_t* launches);

}  // namespace dpk
