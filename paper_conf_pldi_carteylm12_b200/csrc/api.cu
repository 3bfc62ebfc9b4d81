// C ABI (include/dp.h): plan lifecycle, dispatch to the kernels, traceback,
// host-buffer entry point. No exception crosses this boundary.
#include <algorithm>
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <new>
#include <utility>
#include <vector>
#include <cuda_runtime.h>
#include <nvtx3/nvToolsExt.h>

#include "dp.h"
#include "dp_internal.h"

namespace {

struct DevBuf {
  void* ptr = nullptr;
  size_t bytes = 0;
  cudaError_t ensure(size_t want) {
    if (want <= bytes) return cudaSuccess;
    if (ptr) cudaFree(ptr);
    ptr = nullptr;
    bytes = 0;
    cudaError_t e = cudaMalloc(&ptr, want);
    if (e == cudaSuccess) bytes = want;
    return e;
  }
  void release() {
    if (ptr) cudaFree(ptr);
    ptr = nullptr;
    bytes = 0;
  }
};

// NVTX range around an ABI call (header-only NVTX v3: a no-op unless a profiler attaches), so
// nsight timelines show plan / solve / traceback / host-pipeline phases (SURVEY §5 tracing).
struct NvtxRange {
  explicit NvtxRange(const char* name) { nvtxRangePushA(name); }
  ~NvtxRange() { nvtxRangePop(); }
};

// Makes the plan's device current for the lifetime of a call and restores the caller's on every
// exit path (the plan binds the device that was current at dp_plan_create).
struct DeviceGuard {
  int prev = -1;
  explicit DeviceGuard(int dev) {
    if (cudaGetDevice(&prev) != cudaSuccess) prev = -1;
    if (prev != dev) cudaSetDevice(dev);
  }
  ~DeviceGuard() {
    int cur = -1;
    if (prev >= 0 && cudaGetDevice(&cur) == cudaSuccess && cur != prev) cudaSetDevice(prev);
  }
};

}  // namespace

struct dp_plan {
  int kind = 0;
  int device = 0;
  int64_t max_la = 0, max_lb = 0;
  int asz = 0, gap = 0, hairpin = 0, S = 0, K = 0;
  int gap_open = 0, gap_ext = 0;  // DP_SW_AFFINE
  bool want_tb = false;
  int ndim = 2;
  int32_t coeff[DP_MAX_DIM] = {0, 0, 0, 0};
  int64_t p_lo = 0, p_hi = 0;
  int64_t ext[2] = {1, 1};
  int32_t window = -1;
  int32_t cand[24][2] = {};  // DP_DIAG_LCS: §4.7 candidate schedules
  int ncand = 0, force = -1;
  // device parameters
  int8_t* d_sigma = nullptr;
  std::vector<int8_t> h_sigma;
  bool packed16 = false;  // SW on the s16x2 two-problems-per-warp kernels
  bool affine16 = false;  // affine SW on the s16x2 two-problems-per-warp kernel
  bool inter = false;     // SW on the inter-task kernel (one pair per thread; short pairs)
  uint8_t* d_pair = nullptr;
  float *d_pi = nullptr, *d_A = nullptr, *d_E = nullptr;
  int32_t *d_lpi = nullptr, *d_lA = nullptr, *d_lE = nullptr;
  int v16_C = 0, v16_sat = 0;  // Viterbi on the s16x2 kernel when v16_C > 0 (hmm_vit16.cu guard)
  int L = 0;                                         // DP_PROFILE_FORWARD positions
  float *d_ptr = nullptr, *d_pem = nullptr, *d_pei = nullptr;
  // retained state of the most recent solve
  DevBuf tb_state, tb_aux, tb_aux2, scratch;
  DevBuf tb_state_alt;             // host entry point: the other chunk's retained state (packed SW)
  cudaStream_t s_cmp = nullptr;    // host entry point: second compute stream (packed SW)
  int64_t last_n = -1;
  int64_t last_max_la = 0, last_max_lb = 0;
  const uint8_t *last_a = nullptr, *last_b = nullptr;
  const int64_t *last_aoff = nullptr, *last_boff = nullptr;
  int32_t* last_scores = nullptr;  // device (alignment traceback reads the score)
  DevBuf own_scores;               // when the caller's scores are float/host we keep a copy
  // host-API staging (dp_solve_batch_host): copies run on their own streams,
  // chunk by chunk, overlapped with the solve of the neighbouring chunks
  DevBuf h_a, h_b, h_aoff, h_boff, h_scores, h_tb, h_tblen, h_coords;
  cudaStream_t s_h2d = nullptr, s_d2h = nullptr;
  static constexpr int kMaxChunks = 16;
  cudaEvent_t ev_start = nullptr, ev_in[kMaxChunks] = {}, ev_out[kMaxChunks] = {};
  int64_t launches = 0;
  const char* variant = "";  // kernel family of the last solve (dp_plan_last_variant)
  bool vit_walked = false;  // the last Viterbi solve walked its paths into tb_aux2
  // dp_solve: a ring of {0, len_a, 0, len_b} offset slots in device memory; a slot is reused only
  // after the event recorded behind the solve that read it has completed
  static constexpr int kSolveSlots = 16;
  DevBuf solve_off;
  cudaEvent_t solve_ev[kSolveSlots] = {};
  int solve_next = 0;
  // diagnostics (environment, read once at dp_plan_create; tests and experiments only)
  struct {
    bool force_int32 = false, nuss_cell = false, hmm_timing = false, nuss_timing = false, sw_timing = false;
    bool nuss_rounds = false, diag_generic = false, sw_intra = false;
    int64_t nuss_tiled_min = 32;
    int nuss_tbw = 0, diag_force = -1, host_chunks = 0;  // 0: per kind (see dp_solve_batch_host)
    double host_edge = 0.5;  // first / last host chunk size relative to the others (config 2 e2e: 1.0 / 0.5 / 0.3: 2.97 / 2.91 / 2.92 ms)
    bool hmm_simt = false, nuss_no_cluster = false, hmm_separate_walk = false;
    int hmm_ns = 0, hmm_tc_smem_kb = -1;
  } env;
};

namespace {

void read_env(dp_plan* p) {
  auto on = [](const char* k) { return getenv(k) != nullptr; };
  p->env.force_int32 = on("DP_FORCE_INT32");
  p->env.nuss_cell = on("DP_NUSS_CELL");
  p->env.hmm_timing = on("DP_HMM_TIMING");
  p->env.nuss_timing = on("DP_NUSS_TIMING");
  p->env.sw_timing = on("DP_SW_TIMING");
  p->env.nuss_rounds = on("DP_NUSS_ROUNDS");
  p->env.diag_generic = on("DP_DIAG_GENERIC");
  p->env.sw_intra = on("DP_SW_INTRA");
  if (on("DP_NUSS_TILED_MIN")) p->env.nuss_tiled_min = atoll(getenv("DP_NUSS_TILED_MIN"));
  if (on("DP_NUSS_TBW")) p->env.nuss_tbw = atoi(getenv("DP_NUSS_TBW"));
  if (on("DP_DIAG_FORCE")) p->env.diag_force = atoi(getenv("DP_DIAG_FORCE"));
  p->env.hmm_simt = on("DP_HMM_SIMT");
  p->env.nuss_no_cluster = on("DP_NUSS_NO_CLUSTER");
  p->env.hmm_separate_walk = on("DP_HMM_SEPARATE_WALK");
  if (on("DP_HMM_NS")) p->env.hmm_ns = atoi(getenv("DP_HMM_NS"));
  if (on("DP_HMM_TC_SMEM_KB")) p->env.hmm_tc_smem_kb = atoi(getenv("DP_HMM_TC_SMEM_KB"));
  if (on("DP_HOST_EDGE")) p->env.host_edge = std::max(0.05, std::min(1.0, atof(getenv("DP_HOST_EDGE"))));
  if (on("DP_HOST_CHUNKS")) p->env.host_chunks = std::max(1, std::min(dp_plan::kMaxChunks, atoi(getenv("DP_HOST_CHUNKS"))));
}

int max_smem_optin(int dev) {
  int v = 0;
  if (cudaDeviceGetAttribute(&v, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev) != cudaSuccess) v = 0;
  return v;
}

dp_status cuda_status(cudaError_t e) {
  if (e == cudaSuccess) return DP_OK;
  static const bool verbose = getenv("DP_VERBOSE_ERRORS") != nullptr;  // diagnostic: name the CUDA error
  if (verbose) fprintf(stderr, "dp: CUDA error %s: %s\n", cudaGetErrorName(e), cudaGetErrorString(e));
  if (e == cudaErrorMemoryAllocation) return DP_E_NOMEM;
  return DP_E_CUDA;
}

template <typename T>
cudaError_t upload(T** dst, const T* src, size_t count) {
  cudaError_t e = cudaMalloc(reinterpret_cast<void**>(dst), count * sizeof(T));
  if (e != cudaSuccess) return e;
  return cudaMemcpy(*dst, src, count * sizeof(T), cudaMemcpyHostToDevice);
}

// Dependency families of each recurrence, in the index
// order of its definition. Alignment: (i, j); Nussinov: (i, j); HMM: (s, i).
int families(int kind, int64_t la, int64_t lb, int S, int64_t ext[2], int* triangular, dp_dep deps[8]) {
  memset(deps, 0, sizeof(dp_dep) * 8);
  for (int d = 0; d < 8; ++d) deps[d].ranged_axis = -1;
  *triangular = 0;
  switch (kind) {
    case DP_EDIT:
    case DP_SW_LINEAR:  // d(i-1,j), d(i,j-1), d(i-1,j-1)  (Fig.7; §6.1)
    case DP_SW_AFFINE:  // E <- (0,-1), F <- (-1,0), H <- (-1,-1); same-cell H <- E, F orders a cell's tables
      ext[0] = la + 1; ext[1] = lb + 1;
      deps[0].offset[0] = -1;
      deps[1].offset[1] = -1;
      deps[2].offset[0] = -1; deps[2].offset[1] = -1;
      return 3;
    case DP_NUSSINOV: {  // gamma(i+1,j), gamma(i,j-1), gamma(i+1,j-1), gamma(i,k), gamma(k+1,j), i<k<j
      const int64_t n = la > 1 ? la : 2;
      ext[0] = n; ext[1] = n;
      *triangular = 1;
      deps[0].offset[0] = 1;
      deps[1].offset[1] = -1;
      deps[2].offset[0] = 1; deps[2].offset[1] = -1;
      deps[3].ranged_axis = 1; deps[3].lo = -(n - 1); deps[3].hi = -1;  // (0, k - j)
      deps[4].ranged_axis = 0; deps[4].lo = 1; deps[4].hi = n - 1;      // (k + 1 - i, 0)
      return 5;
    }
    case DP_DIAG_LCS:  // f(x-1, y-1) only (§4.7)
      ext[0] = la + 1; ext[1] = lb + 1;
      deps[0].offset[0] = -1; deps[0].offset[1] = -1;
      return 1;
    case DP_PROFILE_FORWARD:  // (j, i): M <- (-1,-1), I <- (0,-1), D <- (-1,0) (position-major state order)
      ext[0] = S + 1; ext[1] = la + 1;
      deps[0].offset[0] = -1; deps[0].offset[1] = -1;
      deps[1].offset[1] = -1;
      deps[2].offset[0] = -1;
      return 3;
    case DP_HMM_FORWARD:
    case DP_HMM_VITERBI:  // F(t.start, i-1) for t in s.transitionsto: any state (§5.2)
      ext[0] = S; ext[1] = la + 1;
      deps[0].offset[1] = -1;
      deps[0].ranged_axis = 0; deps[0].lo = -(S - 1); deps[0].hi = S - 1;
      return 1;
  }
  return -1;
}

// Packed-SW arguments; with traceback the checkpoint buffers live in the plan.
cudaError_t sw16_args(dp_plan* p, int64_t n, const uint8_t* a_cat, const int64_t* a_off, const uint8_t* b_cat,
                      const int64_t* b_off, int64_t max_la, int64_t max_lb, int32_t* scores, dpk::Sw16Args* A) {
  A->n = n; A->a_cat = a_cat; A->b_cat = b_cat; A->a_off = a_off; A->b_off = b_off;
  A->max_la = max_la > 0 ? max_la : 1; A->max_lb = max_lb > 0 ? max_lb : 1;
  A->sigma = p->d_sigma; A->asz = p->asz; A->gap = p->gap;
  A->smem_per_warp = dpk::sw16_smem_per_warp(p->asz, A->max_la, A->max_lb);
  A->scores = scores;
  if (!p->want_tb) return cudaSuccess;
  int64_t strips, nslab, rw, cw, bw;
  dpk::sw16_state_words(n, A->max_la, A->max_lb, &strips, &nslab, &rw, &cw, &bw);
  cudaError_t e = p->tb_state.ensure((size_t)(rw + cw + bw) * 4 + 64);
  if (e != cudaSuccess) return e;
  A->rowck = static_cast<uint32_t*>(p->tb_state.ptr);
  A->colck = A->rowck + rw;
  A->slabbest = A->colck + cw;
  const int64_t slab_words = ((n + 1) / 2) * strips * (nslab > 0 ? nslab : 1) * 32;
  A->corner = A->slabbest + slab_words;
  A->lanebest = A->corner + slab_words;
  A->strips_max = strips;
  A->nslab_max = nslab > 0 ? nslab : 1;
  A->tb_ctr = reinterpret_cast<unsigned long long*>(
      (reinterpret_cast<uintptr_t>(A->rowck + rw + cw + bw) + 15) & ~static_cast<uintptr_t>(15));
  p->last_scores = scores;
  return cudaSuccess;
}

}  // namespace

extern "C" {

int dp_abi_version(void) { return DP_ABI_VERSION; }

const char* dp_status_string(dp_status s) {
  switch (s) {
    case DP_OK: return "ok";
    case DP_E_INVALID: return "invalid argument";
    case DP_E_NO_SCHEDULE: return "no valid schedule (cyclic dependencies)";
    case DP_E_UNSUPPORTED: return "unsupported";
    case DP_E_TOO_LARGE: return "size exceeds plan maximum or device limit";
    case DP_E_NOMEM: return "out of memory";
    case DP_E_CUDA: return "CUDA error";
    case DP_E_NO_TRACEBACK: return "no traceback retained";
  }
  return "unknown status";
}

void dp_plan_destroy(dp_plan_t p) {
  if (!p) return;
  int cur = 0;
  cudaGetDevice(&cur);
  cudaSetDevice(p->device);
  cudaFree(p->d_sigma); cudaFree(p->d_pair);
  cudaFree(p->d_pi); cudaFree(p->d_A); cudaFree(p->d_E);
  cudaFree(p->d_lpi); cudaFree(p->d_lA); cudaFree(p->d_lE);
  cudaFree(p->d_ptr); cudaFree(p->d_pem); cudaFree(p->d_pei);
  DevBuf* bufs[] = {&p->tb_state, &p->tb_aux, &p->tb_aux2, &p->scratch, &p->own_scores, &p->h_a, &p->h_b,
                    &p->h_aoff, &p->h_boff, &p->h_scores, &p->h_tb, &p->h_tblen, &p->h_coords};
  for (DevBuf* b : bufs) b->release();
  if (p->s_h2d) cudaStreamDestroy(p->s_h2d);
  if (p->s_cmp) cudaStreamDestroy(p->s_cmp);
  p->tb_state_alt.release();
  p->solve_off.release();
  for (int k = 0; k < dp_plan::kSolveSlots; ++k)
    if (p->solve_ev[k]) cudaEventDestroy(p->solve_ev[k]);
  if (p->s_d2h) cudaStreamDestroy(p->s_d2h);
  if (p->ev_start) cudaEventDestroy(p->ev_start);
  for (int k = 0; k < dp_plan::kMaxChunks; ++k) {
    if (p->ev_in[k]) cudaEventDestroy(p->ev_in[k]);
    if (p->ev_out[k]) cudaEventDestroy(p->ev_out[k]);
  }
  cudaSetDevice(cur);
  delete p;
}

dp_status dp_plan_create(const dp_desc* d, dp_plan_t* out) {
  NvtxRange nvtx("dp_plan_create");
  if (!d || !out) return DP_E_INVALID;
  *out = nullptr;
  if (d->struct_size != sizeof(dp_desc)) return DP_E_INVALID;
  if (d->kind < DP_EDIT || d->kind > DP_PROFILE_FORWARD) return DP_E_INVALID;
  if (d->max_len_a < 0 || d->max_len_b < 0) return DP_E_INVALID;
  dp_plan* p = new (std::nothrow) dp_plan();
  if (!p) return DP_E_NOMEM;
  p->kind = d->kind;
  p->max_la = d->max_len_a;
  p->max_lb = d->max_len_b;
  p->want_tb = d->want_traceback != 0;
  cudaGetDevice(&p->device);
  read_env(p);
  const int smem_limit = max_smem_optin(p->device);
  dp_status st = DP_OK;
  cudaError_t e = cudaSuccess;
  switch (d->kind) {
    case DP_EDIT:
      p->asz = d->alphabet_size > 0 ? d->alphabet_size : 32;
      if (p->asz > 32) st = DP_E_UNSUPPORTED;
      p->gap = 1;
      if (d->max_len_b > (1 << 20) || d->max_len_a > (1 << 20)) st = DP_E_TOO_LARGE;
      // the warp kernel keeps the column residues (and the strip boundary row) in shared memory
      else if (smem_limit > 0 && dpk::align_smem_bytes(p->asz, false, d->max_len_a, d->max_len_b) > (size_t)smem_limit)
        st = DP_E_TOO_LARGE;
      break;
    case DP_SW_LINEAR:
      p->asz = d->alphabet_size;
      if (!d->sigma || p->asz < 1 || d->gap <= 0) { st = DP_E_INVALID; break; }
      if (p->asz > 32) { st = DP_E_UNSUPPORTED; break; }
      p->gap = d->gap;
      if (d->max_len_b > (1 << 20) || d->max_len_a > (1 << 20)) { st = DP_E_TOO_LARGE; break; }
      e = upload(&p->d_sigma, d->sigma, (size_t)p->asz * p->asz);
      p->h_sigma.assign(d->sigma, d->sigma + (size_t)p->asz * p->asz);
      // hybrid dispatch (§6.1): short pairs one per thread (inter-task), longer ones on the
      // warp kernels (intra-task); DP_SW_INTRA=1 keeps short pairs on the warp kernels (comparison)
      p->inter = dpk::sw_inter_eligible(d->max_len_a, d->max_len_b, p->asz, p->gap) && !p->env.sw_intra;
      p->packed16 = !p->inter && dpk::sw16_eligible(d->max_len_a, d->max_len_b, d->sigma, p->asz, p->gap, d->want_traceback != 0) &&
                    !p->env.force_int32 &&
                    (smem_limit <= 0 || dpk::sw16_smem_bytes(p->asz, d->max_len_a, d->max_len_b) <= (size_t)smem_limit);
      if (!p->inter && !p->packed16 && smem_limit > 0 &&
          dpk::align_smem_bytes(p->asz, true, d->max_len_a, d->max_len_b) > (size_t)smem_limit)
        st = DP_E_TOO_LARGE;
      break;
    case DP_SW_AFFINE:
      p->asz = d->alphabet_size;
      if (!d->sigma || p->asz < 1 || d->gap_open < 0 || d->gap_extend < 1) { st = DP_E_INVALID; break; }
      if (p->asz > 32) { st = DP_E_UNSUPPORTED; break; }
      p->gap_open = d->gap_open; p->gap_ext = d->gap_extend;
      if (d->max_len_b > (1 << 20) || d->max_len_a > (1 << 20)) { st = DP_E_TOO_LARGE; break; }
      p->affine16 = dpk::affine16_eligible(d->max_len_a, d->max_len_b, d->sigma, p->asz, p->gap_open, p->gap_ext) &&
                    !p->env.force_int32 &&
                    (smem_limit <= 0 || dpk::affine16_smem_bytes(p->asz, d->max_len_a, d->max_len_b) <= (size_t)smem_limit);
      if (!p->affine16 && smem_limit > 0 &&
          dpk::align_affine_smem_bytes(p->asz, d->max_len_a, d->max_len_b) > (size_t)smem_limit) {
        st = DP_E_TOO_LARGE;
        break;
      }
      e = upload(&p->d_sigma, d->sigma, (size_t)p->asz * p->asz);
      p->h_sigma.assign(d->sigma, d->sigma + (size_t)p->asz * p->asz);
      break;
    case DP_DIAG_LCS:
      if (p->want_tb) { st = DP_E_UNSUPPORTED; break; }
      p->asz = d->alphabet_size > 0 && d->alphabet_size <= 256 ? d->alphabet_size : 0;  // optional
      if (d->max_len_a > 40000 || d->max_len_b > 40000) st = DP_E_TOO_LARGE;  // uint16 window rows in smem
      else if (smem_limit > 0 &&
               dpk::diag_smem_bytes(std::max(d->max_len_a, d->max_len_b), p->asz) > (size_t)smem_limit)
        st = DP_E_TOO_LARGE;
      break;
    case DP_NUSSINOV:
      if (!d->pair_mask || d->min_hairpin < 0) { st = DP_E_INVALID; break; }
      if (d->max_len_a > 32767 * 2) { st = DP_E_TOO_LARGE; break; }
      p->hairpin = d->min_hairpin;
      e = upload(&p->d_pair, d->pair_mask, 16);
      break;
    case DP_PROFILE_FORWARD:
      p->L = d->n_positions;
      p->K = d->alphabet_size;
      if (p->L < 1 || p->K < 1 || !d->ptrans || !d->pemit_m || !d->pemit_i) { st = DP_E_INVALID; break; }
      if (p->K > 32) { st = DP_E_UNSUPPORTED; break; }
      if (p->want_tb) { st = DP_E_UNSUPPORTED; break; }
      if (smem_limit > 0 && dpk::phmm_smem_bytes(p->L, p->K, d->max_len_a) > (size_t)smem_limit) {
        st = DP_E_TOO_LARGE;
        break;
      }
      p->S = p->L;
      e = upload(&p->d_ptr, d->ptrans, (size_t)(p->L + 1) * 9);
      if (e == cudaSuccess) e = upload(&p->d_pem, d->pemit_m, (size_t)(p->L + 1) * p->K);
      if (e == cudaSuccess) e = upload(&p->d_pei, d->pemit_i, (size_t)(p->L + 1) * p->K);
      break;
    case DP_HMM_FORWARD:
    case DP_HMM_VITERBI:
      p->S = d->n_states;
      p->K = d->alphabet_size;
      if (p->S < 1 || p->K < 1) { st = DP_E_INVALID; break; }
      if (p->S > 64 || p->K > 16) { st = DP_E_UNSUPPORTED; break; }
      if (d->kind == DP_HMM_FORWARD) {
        if (!d->pi || !d->A || !d->E) { st = DP_E_INVALID; break; }
        if (p->want_tb) { st = DP_E_UNSUPPORTED; break; }
        e = upload(&p->d_pi, d->pi, p->S);
        if (e == cudaSuccess) e = upload(&p->d_A, d->A, (size_t)p->S * p->S);
        if (e == cudaSuccess) e = upload(&p->d_E, d->E, (size_t)p->S * p->K);
      } else {
        if (!d->lpi || !d->lA || !d->lE) { st = DP_E_INVALID; break; }
        e = upload(&p->d_lpi, d->lpi, p->S);
        if (e == cudaSuccess) e = upload(&p->d_lA, d->lA, (size_t)p->S * p->S);
        if (e == cudaSuccess) e = upload(&p->d_lE, d->lE, (size_t)p->S * p->K);
        // exact in 16 bits for these scores? (DP_FORCE_INT32: the int32 kernel regardless)
        if (!p->env.force_int32) p->v16_C = dpk::vit16_clamp(d->lA, d->lE, p->S, p->K, &p->v16_sat);
      }
      break;
  }
  if (st == DP_OK && e != cudaSuccess) st = cuda_status(e);
  if (st == DP_OK) {
    // schedule (A1–A4): derive, or verify the user's
    int tri = 0;
    dp_dep deps[8];
    int nd = families(d->kind, p->max_la, p->max_lb, p->S, p->ext, &tri, deps);
    p->ndim = 2;
    st = dp_schedule_derive(2, p->ext, tri, nd, deps, d->coeff_bound, d->user_coeff, p->coeff, &p->p_lo, &p->p_hi,
                            &p->window);
    if (st == DP_OK && d->kind == DP_DIAG_LCS) {
      // §4.7: every candidate schedule; the kernel picks one per problem. A (valid) user
      // schedule must be one of them and is then used for every problem.
      int32_t c[24 * 2];
      st = dp_schedule_conditional(2, nd, deps, d->coeff_bound, 24, c, &p->ncand);
      for (int k = 0; st == DP_OK && k < p->ncand; ++k) {
        p->cand[k][0] = c[2 * k]; p->cand[k][1] = c[2 * k + 1];
        if (d->user_coeff && c[2 * k] == d->user_coeff[0] && c[2 * k + 1] == d->user_coeff[1]) p->force = k;
      }
      if (st == DP_OK && d->user_coeff && p->force < 0) st = DP_E_UNSUPPORTED;
    }
  }
  if (st == DP_OK && d->kind != DP_DIAG_LCS) {
    // The kernels implement the derived schedule; a user schedule that is valid
    // but differs would need another kernel (conditional schedules, §4.7: NEXT).
    // Coefficients of a dimension of extent 1 do not change the partitions.
    static const int32_t expect[8][2] = {{1, 1}, {1, 1}, {-1, 1}, {0, 1}, {0, 1}, {1, 1}, {0, 0}, {1, 1}};
    for (int i = 0; i < 2; ++i)
      if (p->ext[i] > 1 && p->coeff[i] != expect[d->kind][i]) st = DP_E_UNSUPPORTED;
  }
  if (st != DP_OK) {
    dp_plan_destroy(p);
    return st;
  }
  *out = p;
  return DP_OK;
}

dp_status dp_plan_get_schedule(dp_plan_t p, int32_t coeff[], int* ndim, int64_t* p_lo, int64_t* p_hi,
                               int32_t* window) {
  if (!p) return DP_E_INVALID;
  if (coeff) for (int i = 0; i < p->ndim; ++i) coeff[i] = p->coeff[i];
  if (ndim) *ndim = p->ndim;
  if (p_lo) *p_lo = p->p_lo;
  if (p_hi) *p_hi = p->p_hi;
  if (window) *window = p->window;
  return DP_OK;
}

int64_t dp_plan_launch_count(dp_plan_t p) { return p ? p->launches : -1; }
const char* dp_plan_last_variant(dp_plan_t p) { return p ? p->variant : ""; }

dp_status dp_solve_batch(dp_plan_t p, int64_t n, const uint8_t* a_cat, const int64_t* a_off, const uint8_t* b_cat,
                         const int64_t* b_off, int64_t max_len_a, int64_t max_len_b, void* scores_out,
                         void* stream) {
  NvtxRange nvtx("dp_solve_batch");
  if (!p || n < 0) return DP_E_INVALID;
  if (n > 0 && (!a_off || !scores_out)) return DP_E_INVALID;
  const bool align =
      p->kind == DP_EDIT || p->kind == DP_SW_LINEAR || p->kind == DP_SW_AFFINE || p->kind == DP_DIAG_LCS;
  if (align && n > 0 && !b_off) return DP_E_INVALID;
  if (max_len_a < 0 || max_len_b < 0) return DP_E_INVALID;
  if (max_len_a > p->max_la || (align && max_len_b > p->max_lb)) return DP_E_TOO_LARGE;
  cudaStream_t s = reinterpret_cast<cudaStream_t>(stream);
  DeviceGuard guard(p->device);
  cudaError_t e = cudaSuccess;
  p->last_n = n;
  p->last_a = a_cat; p->last_b = b_cat; p->last_aoff = a_off; p->last_boff = b_off;
  p->last_max_la = max_len_a; p->last_max_lb = max_len_b;
  switch (p->kind) {
    case DP_DIAG_LCS: {
      dpk::DiagArgs A{};
      A.n = n; A.a_cat = a_cat; A.b_cat = b_cat; A.a_off = a_off; A.b_off = b_off;
      A.max_len = std::max<int64_t>(1, std::max(max_len_a, max_len_b));
      A.scores = static_cast<int32_t*>(scores_out);
      A.ncand = p->ncand;
      for (int k = 0; k < p->ncand; ++k) { A.cand[k][0] = p->cand[k][0]; A.cand[k][1] = p->cand[k][1]; }
      A.force = p->env.diag_force >= 0 ? p->env.diag_force : p->force;  // env: diagnostic
      A.asz = p->env.diag_generic ? 0 : p->asz;  // env: diagnostic (the unpacked path)
      p->variant = "k_diag";
      e = dpk::diag_solve(A, s, &p->launches);
      break;
    }
    case DP_SW_LINEAR:
      if (p->inter) {
        dpk::AlignArgs A{};
        A.n = n; A.a_cat = a_cat; A.b_cat = b_cat; A.a_off = a_off; A.b_off = b_off;
        A.max_la = max_len_a; A.max_lb = max_len_b;
        A.sigma = p->d_sigma; A.asz = p->asz; A.gap = p->gap; A.local = true;
        A.scores = static_cast<int32_t*>(scores_out);
        if (p->want_tb) {
          A.dir_stride = dpk::sw_inter_dir_words(p->max_la);
          e = p->tb_state.ensure((size_t)(n * A.dir_stride * 4 + 16));
          if (e == cudaSuccess) e = p->tb_aux.ensure((size_t)(n * 2 * 4 + 16));
          if (e != cudaSuccess) break;
          A.dirs = static_cast<uint32_t*>(p->tb_state.ptr);
          A.ends = static_cast<int32_t*>(p->tb_aux.ptr);
          p->last_scores = A.scores;
        }
        e = p->scratch.ensure(dpk::sw_inter_work_bytes(n));
        p->variant = "k_sw_inter";
        if (e == cudaSuccess) e = dpk::sw_inter_solve(A, p->scratch.ptr, s, &p->launches);
        break;
      }
      if (p->packed16) {
        dpk::Sw16Args A{};
        e = sw16_args(p, n, a_cat, a_off, b_cat, b_off, max_len_a, max_len_b, static_cast<int32_t*>(scores_out), &A);
        p->variant = "k_sw16";
        if (e == cudaSuccess) e = dpk::sw16_solve(A, p->want_tb, s, &p->launches);
        break;
      }
      /* fall through */
    case DP_EDIT: {
      dpk::AlignArgs A{};
      A.n = n; A.a_cat = a_cat; A.b_cat = b_cat; A.a_off = a_off; A.b_off = b_off;
      A.max_la = max_len_a > 0 ? max_len_a : 1; A.max_lb = max_len_b > 0 ? max_len_b : 1;
      A.sigma = p->d_sigma; A.asz = p->asz; A.gap = p->gap; A.local = p->kind == DP_SW_LINEAR;
      A.scores = static_cast<int32_t*>(scores_out);
      if (p->want_tb) {
        A.dir_stride = dpk::align_dir_words(A.max_la, A.max_lb);
        e = p->tb_state.ensure((size_t)(n * A.dir_stride * 4 + 16));
        if (e == cudaSuccess) e = p->tb_aux.ensure((size_t)(n * 2 * 4 + 16));
        if (e != cudaSuccess) break;
        A.dirs = static_cast<uint32_t*>(p->tb_state.ptr);
        A.ends = static_cast<int32_t*>(p->tb_aux.ptr);
        p->last_scores = A.scores;
      }
      p->variant = "k_align";
      e = dpk::align_solve(A, s, &p->launches);
      break;
    }
    case DP_SW_AFFINE: {
      dpk::AlignArgs A{};
      A.n = n; A.a_cat = a_cat; A.b_cat = b_cat; A.a_off = a_off; A.b_off = b_off;
      A.max_la = max_len_a > 0 ? max_len_a : 1; A.max_lb = max_len_b > 0 ? max_len_b : 1;
      A.sigma = p->d_sigma; A.asz = p->asz; A.local = true;
      A.gap_open = p->gap_open; A.gap_ext = p->gap_ext;
      A.scores = static_cast<int32_t*>(scores_out);
      if (p->want_tb) {
        // packed: codes per group of two problems; else per problem
        A.dir_stride = p->affine16 ? dpk::affine16_dir_words(A.max_la, A.max_lb) : dpk::align_affine_dir_words(A.max_la, A.max_lb);
        const int64_t units = p->affine16 ? (n + 1) / 2 : n;
        e = p->tb_state.ensure((size_t)(units * A.dir_stride * 4 + 16));
        if (e == cudaSuccess) e = p->tb_aux.ensure((size_t)(n * 2 * 4 + 16));
        if (e != cudaSuccess) break;
        A.dirs = static_cast<uint32_t*>(p->tb_state.ptr);
        A.ends = static_cast<int32_t*>(p->tb_aux.ptr);
        p->last_scores = A.scores;
      }
      p->variant = p->affine16 ? "k_affine16" : "k_align_affine";
      e = p->affine16 ? dpk::affine16_solve(A, s, &p->launches) : dpk::align_affine_solve(A, s, &p->launches);
      break;
    }
    case DP_NUSSINOV: {
      dpk::NussArgs A{};
      A.n = n; A.x_cat = a_cat; A.x_off = a_off; A.max_len = max_len_a > 0 ? max_len_a : 1;
      A.pair_mask = p->d_pair; A.hairpin = p->hairpin;
      A.scores = static_cast<int32_t*>(scores_out);
      if (p->want_tb) {
        A.db_stride = A.max_len;
        e = p->tb_state.ensure((size_t)(n * A.db_stride + 16));
        if (e == cudaSuccess) e = p->tb_aux.ensure((size_t)(n * 4 + 16));
        if (e != cudaSuccess) break;
        A.db = static_cast<uint8_t*>(p->tb_state.ptr);
        A.db_len = static_cast<int32_t*>(p->tb_aux.ptr);
      }
      // cell-level CTA kernel (table in shared memory) for short sequences, tiled
      // max-plus kernels above (SURVEY §8(a) A6b'); DP_NUSS_CELL=1 forces the cell level
      // (config 1, n = 64: tiled 0.097 ms per step vs 0.109 cell-level)
      // latency regime (config 1: a few problems of <= 128 nt): one CTA per problem, table and
      // traceback in shared memory, one barrier per partition (DP_NUSS_CELL / DP_NUSS_TILED_MIN: the
      // other paths, for comparison)
      if (dpk::nuss_small_supported(A.max_len, n, p->device) && !p->env.nuss_cell && p->env.nuss_tiled_min == 32) {
        p->variant = "k_nuss_small";
        unsigned long long* dbg = nullptr;
        if (p->env.nuss_timing) cudaMalloc(&dbg, 64), cudaMemset(dbg, 0, 64), A.dbg = dbg;
        e = dpk::nuss_small_solve(A, s, &p->launches);
        if (dbg) {  // diagnostic: CTA 0 thread 0 cycles (summed over problems): setup, fill, traceback
          unsigned long long h[3];
          cudaStreamSynchronize(s);
          cudaMemcpy(h, dbg, sizeof(h), cudaMemcpyDeviceToHost);
          fprintf(stderr, "nuss_small cycles: setup %llu fill %llu traceback %llu\n", h[0], h[1], h[2]);
          cudaFree(dbg);
        }
        break;
      }
      // a few mid-length problems: one thread-block cluster each, the table in distributed shared
      // memory (DP_NUSS_NO_CLUSTER: the batch / grid kernels, for comparison)
      if (dpk::nuss_cluster_supported(A.max_len, n, p->device) && !p->env.nuss_cell && !p->env.nuss_no_cluster &&
          p->env.nuss_tiled_min == 32) {
        A.scratch_bytes = dpk::nuss_cluster_scratch_bytes(A.max_len, n);
        e = p->scratch.ensure((size_t)A.scratch_bytes);
        if (e != cudaSuccess) break;
        A.scratch = p->scratch.ptr;
        unsigned long long* rounds = nullptr;
        if (p->env.nuss_rounds) cudaMalloc(&rounds, 8 * 4096), cudaMemset(rounds, 0, 8 * 4096), A.round_ns = rounds;
        unsigned long long* dbg = nullptr;
        if (p->env.nuss_timing) cudaMalloc(&dbg, 64), cudaMemset(dbg, 0, 64), A.dbg = dbg;
        p->variant = "k_nuss_cluster";
        e = dpk::nuss_cluster_solve(A, s, &p->launches);
        if (dbg) {  // diagnostic: cluster-kernel phase cycles summed over warps (stderr)
          unsigned long long h[8];
          cudaStreamSynchronize(s);
          cudaMemcpy(h, dbg, sizeof(h), cudaMemcpyDeviceToHost);
          fprintf(stderr, "cluster: staging %llu micro %llu setupB %llu wavefront %llu records %llu | tiles %llu ksteps %llu\n",
                  h[0], h[1], h[2], h[3], h[4], h[5], h[6]);
          cudaFree(dbg);
        }
        if (rounds) {  // diagnostic: per tile-diagonal [products, finish] durations of cluster 0 (stderr)
          static unsigned long long h[4096];
          cudaStreamSynchronize(s);
          cudaMemcpy(h, rounds, sizeof(h), cudaMemcpyDeviceToHost);
          const int nt = (int)((A.max_len + 31) / 32);
          for (int d = 0; d + 1 < nt; ++d)
            fprintf(stderr, "cluster round %d %.1f us (split-K products %.1f us)\n", d, (h[2 * d + 2] - h[2 * d]) * 1e-3,
                    h[2 * d + 1] ? (h[2 * d + 1] - h[2 * d]) * 1e-3 : 0.0);
          cudaFree(rounds);
        }
        break;
      }
      const bool tiled = A.max_len > p->env.nuss_tiled_min && !p->env.nuss_cell && (n == 1 || A.max_len <= 4096);
      A.scratch_bytes = tiled ? dpk::nuss_tiled_scratch_bytes(A.max_len, n, p->device)
                              : dpk::nuss_scratch_bytes(A.max_len, n, p->device);
      e = p->scratch.ensure((size_t)A.scratch_bytes);
      if (e != cudaSuccess) break;
      A.scratch = p->scratch.ptr;
      unsigned long long* rounds = nullptr;
      A.tbw = p->env.nuss_tbw;
      if (p->env.nuss_rounds && tiled && n == 1) cudaMalloc(&rounds, 8 * 8192), cudaMemset(rounds, 0, 8 * 8192), A.round_ns = rounds;
      unsigned long long* dbg = nullptr;
      if (p->env.nuss_timing && tiled) cudaMalloc(&dbg, 64), cudaMemset(dbg, 0, 64), A.dbg = dbg;
      p->variant = !tiled ? "k_nuss_cell" : (n == 1 && A.max_len > 1024) ? "k_nuss_grid2" : "k_nuss_batch";
      e = tiled ? dpk::nuss_tiled_solve(A, s, &p->launches) : dpk::nuss_solve(A, s, &p->launches);
      if (dbg) {  // diagnostic: batch-kernel phase cycles summed over warps (stderr)
        unsigned long long h[8];
        cudaStreamSynchronize(s);
        cudaMemcpy(h, dbg, sizeof(h), cudaMemcpyDeviceToHost);
        const char* nm[8] = {"stage", "phaseA", "stageB", "wavefront", "records", "score", "traceback", "-"};
        double tot = 0;
        for (int q = 0; q < 7; ++q) tot += (double)h[q];
        for (int q = 0; q < 7; ++q) fprintf(stderr, "nuss %-9s %16llu %5.1f%%\n", nm[q], h[q], 100.0 * h[q] / (tot > 0 ? tot : 1));
        cudaFree(dbg);
      }
      if (rounds) {  // diagnostic: per tile-diagonal round durations of the grid sweep (stderr)
        static unsigned long long h[8192];
        cudaStreamSynchronize(s);
        cudaMemcpy(h, rounds, sizeof(h), cudaMemcpyDeviceToHost);
        const int nt = (int)((A.max_len + 31) / 32);
        for (int d = 0; d + 1 < nt; ++d) fprintf(stderr, "round %d %.1f us\n", d, (h[d + 1] - h[d]) * 1e-3);
        fprintf(stderr, "last round + score %.1f us\n", (h[nt] - h[nt - 1]) * 1e-3);
        if (h[nt + 1] > h[nt]) fprintf(stderr, "traceback %.1f us\n", (h[nt + 1] - h[nt]) * 1e-3);
        fprintf(stderr, "traceback warps: max %llu cycles, sum %llu cycles, %llu intervals, %llu steps\n", h[nt + 2],
                h[nt + 3], h[nt + 4], h[nt + 5]);
        cudaFree(rounds);
      }
      break;
    }
    case DP_PROFILE_FORWARD: {
      dpk::PhmmArgs P{};
      P.n = n; P.x_cat = a_cat; P.x_off = a_off; P.max_len = max_len_a; P.L = p->L; P.K = p->K;
      P.trans = p->d_ptr; P.emit_m = p->d_pem; P.emit_i = p->d_pei;
      P.ll_out = static_cast<float*>(scores_out);
      p->variant = "k_phmm_forward";
      e = dpk::phmm_forward(P, s, &p->launches);
      break;
    }
    case DP_HMM_FORWARD:
    case DP_HMM_VITERBI: {
      dpk::HmmArgs H{};
      H.ns_override = p->env.hmm_ns;
      H.n = n; H.x_cat = a_cat; H.x_off = a_off; H.max_len = max_len_a; H.S = p->S; H.K = p->K;
      if (p->kind == DP_HMM_FORWARD) {
        H.pi = p->d_pi; H.A = p->d_A; H.E = p->d_E;
        H.ll_out = static_cast<float*>(scores_out);
        // the [batch x S] x [S x S] step on tcgen05 (SIMT fallback kernel via DP_HMM_SIMT=1)
        unsigned long long* dbg = nullptr;
        if (p->env.hmm_timing) cudaMalloc(&dbg, 8 * 4 * 66), cudaMemset(dbg, 0, 8 * 4 * 66), H.dbg = dbg;
        H.tc_smem_kb = p->env.hmm_tc_smem_kb;
        const bool tc = dpk::hmm_forward_tc_supported(p->S) && !p->env.hmm_simt;
        p->variant = tc ? "k_forward_tc" : "k_forward";
        e = tc ? dpk::hmm_forward_tc(H, s, &p->launches) : dpk::hmm_forward(H, s, &p->launches);
        if (dbg) {  // diagnostic: CTA 0 step phases (ns): MMA issue, wait for MMA, epilogue, barrier
          unsigned long long h[4 * 66];
          cudaStreamSynchronize(s);
          cudaMemcpy(h, dbg, sizeof(h), cudaMemcpyDeviceToHost);
          double acc[4] = {0, 0, 0, 0};
          int cnt = 0;
          for (int i = 10; i < 65; ++i) {
            if (!h[4 * i] || !h[4 * (i + 1)]) continue;
            acc[0] += h[4 * i + 1] - h[4 * i]; acc[1] += h[4 * i + 2] - h[4 * i + 1];
            acc[2] += h[4 * i + 3] - h[4 * i + 2]; acc[3] += h[4 * (i + 1)] - h[4 * i + 3];
            ++cnt;
          }
          if (cnt) fprintf(stderr, "forward step ns: issue %.0f wait %.0f epilogue %.0f barrier %.0f\n", acc[0] / cnt,
                           acc[1] / cnt, acc[2] / cnt, acc[3] / cnt);
          cudaFree(dbg);
        }
      } else {
        H.lpi = p->d_lpi; H.lA = p->d_lA; H.lE = p->d_lE;
        H.vit_out = static_cast<int32_t*>(scores_out);
        // the s16x2 kernel (two sequences per register, the argmax recovered by its fused walk);
        // the int32 kernel when the scores do not fit or the walk is asked for as its own kernel
        const bool v16 = p->v16_C > 0 && !(p->want_tb && p->env.hmm_separate_walk);
        if (v16) {
          H.v16_C = p->v16_C;
          H.v16_sat = p->v16_sat;
          if (p->want_tb) {
            const int64_t ml = max_len_a > 0 ? max_len_a : 1;
            e = p->tb_state.ensure((size_t)(((n + 1) / 2) * ml * 64 * 4 + 16));
            if (e == cudaSuccess) e = p->tb_aux.ensure((size_t)(n * 4 + 16));
            if (e == cudaSuccess) e = p->tb_aux2.ensure((size_t)(n * ml + 16));
            if (e != cudaSuccess) break;
            H.rows16 = static_cast<uint32_t*>(p->tb_state.ptr);
            H.final_state = static_cast<int32_t*>(p->tb_aux.ptr);
            H.path = static_cast<uint8_t*>(p->tb_aux2.ptr);
            p->vit_walked = true;
          }
          p->variant = "k_viterbi16";
          e = dpk::hmm_viterbi16(H, s, &p->launches);
          break;
        }
        if (p->want_tb) {
          e = p->tb_state.ensure((size_t)(n * (max_len_a > 0 ? max_len_a : 1) * 64 + 16));
          if (e == cudaSuccess) e = p->tb_aux.ensure((size_t)(n * 4 + 16));
          if (e != cudaSuccess) break;
          H.bp = static_cast<uint8_t*>(p->tb_state.ptr);
          H.final_state = static_cast<int32_t*>(p->tb_aux.ptr);
          // the paths, walked inside k_viterbi right behind the sweep (DP_HMM_SEPARATE_WALK: the
          // walk as its own kernel at dp_traceback, for comparison)
          if (!p->env.hmm_separate_walk) {
            e = p->tb_aux2.ensure((size_t)(n * (max_len_a > 0 ? max_len_a : 1) + 16));
            if (e != cudaSuccess) break;
            H.path = static_cast<uint8_t*>(p->tb_aux2.ptr);
          }
          p->vit_walked = H.path != nullptr;
        }
        p->variant = "k_viterbi";
        e = dpk::hmm_viterbi(H, s, &p->launches);
      }
      break;
    }
  }
  if (e != cudaSuccess) {
    p->last_n = -1;
    return cuda_status(e);
  }
  return DP_OK;
}

dp_status dp_solve(dp_plan_t p, const uint8_t* a, int64_t len_a, const uint8_t* b, int64_t len_b, void* score_out,
                   void* stream) {
  if (!p || len_a < 0 || len_b < 0 || !score_out) return DP_E_INVALID;
  const bool align =
      p->kind == DP_EDIT || p->kind == DP_SW_LINEAR || p->kind == DP_SW_AFFINE || p->kind == DP_DIAG_LCS;
  if ((len_a > 0 && !a) || (align && len_b > 0 && !b)) return DP_E_INVALID;
  if (len_a > p->max_la || (align && len_b > p->max_lb)) return DP_E_TOO_LARGE;
  DeviceGuard guard(p->device);
  cudaStream_t s = reinterpret_cast<cudaStream_t>(stream);
  // offsets {0, len_a, 0, len_b} in a slot of the plan's ring; the slot's previous reader has
  // finished once its event has (host wait, normally long done), so calls on different streams
  // never share a live slot
  cudaError_t e = p->solve_off.ensure(dp_plan::kSolveSlots * 32);
  const int slot = p->solve_next;
  if (e == cudaSuccess && !p->solve_ev[slot]) e = cudaEventCreateWithFlags(&p->solve_ev[slot], cudaEventDisableTiming);
  if (e == cudaSuccess) e = cudaEventSynchronize(p->solve_ev[slot]);
  if (e != cudaSuccess) return cuda_status(e);
  int64_t* d = static_cast<int64_t*>(p->solve_off.ptr) + 4 * slot;
  const int64_t off[4] = {0, len_a, 0, len_b};
  e = cudaMemcpyAsync(d, off, sizeof(off), cudaMemcpyHostToDevice, s);
  if (e != cudaSuccess) return cuda_status(e);
  const dp_status st = dp_solve_batch(p, 1, a, d, align ? b : nullptr, align ? d + 2 : nullptr, len_a,
                                      align ? len_b : 0, score_out, stream);
  e = cudaEventRecord(p->solve_ev[slot], s);
  p->solve_next = (slot + 1) % dp_plan::kSolveSlots;
  if (st != DP_OK) return st;
  return cuda_status(e);
}

dp_status dp_traceback(dp_plan_t p, int64_t first, int64_t count, uint8_t* out, int64_t stride, int32_t* out_len,
                       int32_t* coords, void* stream) {
  NvtxRange nvtx("dp_traceback");
  if (!p) return DP_E_INVALID;
  if (p->kind == DP_HMM_FORWARD || p->kind == DP_PROFILE_FORWARD) return DP_E_UNSUPPORTED;
  if (!p->want_tb || p->last_n < 0) return DP_E_NO_TRACEBACK;
  if (first < 0 || count < 0 || first + count > p->last_n || stride < 0) return DP_E_INVALID;
  if (count > 0 && (!out || !out_len)) return DP_E_INVALID;
  cudaStream_t s = reinterpret_cast<cudaStream_t>(stream);
  DeviceGuard guard(p->device);
  cudaError_t e = cudaSuccess;
  switch (p->kind) {
    case DP_SW_LINEAR:
      if (p->inter) {
        if (stride < p->last_max_la + p->last_max_lb) return DP_E_TOO_LARGE;
        dpk::AlignArgs A{};
        A.n = p->last_n; A.a_cat = p->last_a; A.b_cat = p->last_b; A.a_off = p->last_aoff; A.b_off = p->last_boff;
        A.scores = p->last_scores;
        A.sigma = p->d_sigma; A.asz = p->asz; A.gap = p->gap;
        A.dirs = static_cast<uint32_t*>(p->tb_state.ptr);
        A.dir_stride = dpk::sw_inter_dir_words(p->max_la);
        A.ends = static_cast<int32_t*>(p->tb_aux.ptr);
        e = dpk::sw_inter_traceback(A, p->scratch.ptr, first, count, out, stride, out_len, coords, s, &p->launches);
        break;
      }
      if (p->packed16) {
        if (stride < p->last_max_la + p->last_max_lb) return DP_E_TOO_LARGE;
        dpk::Sw16Args A{};
        e = sw16_args(p, p->last_n, p->last_a, p->last_aoff, p->last_b, p->last_boff, p->last_max_la,
                      p->last_max_lb, p->last_scores, &A);
        unsigned long long* dbg = nullptr;
        if (p->env.sw_timing) cudaMalloc(&dbg, 64), cudaMemset(dbg, 0, 64), A.dbg = dbg;
        if (e == cudaSuccess) e = dpk::sw16_traceback(A, first, count, out, stride, out_len, coords, s, &p->launches);
        if (dbg) {  // diagnostic: traceback phase cycles summed over warps
          unsigned long long h[8];
          cudaStreamSynchronize(s);
          cudaMemcpy(h, dbg, sizeof(h), cudaMemcpyDeviceToHost);
          const char* nm[8] = {"prologue", "probe", "setup", "recompute", "search", "walk", "output", "rounds"};
          double tot = 0;
          for (int q = 0; q < 7; ++q) tot += (double)h[q];
          for (int q = 0; q < 8; ++q) fprintf(stderr, "tb %-9s %14llu %5.1f%%\n", nm[q], h[q], q < 7 ? 100.0 * h[q] / tot : 0.0);
          cudaFree(dbg);
        }
        break;
      }
      /* fall through */
    case DP_EDIT: {
      if (stride < p->last_max_la + p->last_max_lb) return DP_E_TOO_LARGE;
      dpk::AlignArgs A{};
      A.n = p->last_n; A.a_cat = p->last_a; A.b_cat = p->last_b; A.a_off = p->last_aoff; A.b_off = p->last_boff;
      A.max_la = p->last_max_la > 0 ? p->last_max_la : 1; A.max_lb = p->last_max_lb > 0 ? p->last_max_lb : 1;
      A.sigma = p->d_sigma; A.asz = p->asz; A.gap = p->gap; A.local = p->kind == DP_SW_LINEAR;
      A.scores = p->last_scores;
      A.dirs = static_cast<uint32_t*>(p->tb_state.ptr);
      A.dir_stride = dpk::align_dir_words(A.max_la, A.max_lb);
      A.ends = static_cast<int32_t*>(p->tb_aux.ptr);
      e = dpk::align_traceback(A, first, count, out, stride, out_len, coords, s, &p->launches);
      break;
    }
    case DP_SW_AFFINE: {
      if (stride < p->last_max_la + p->last_max_lb) return DP_E_TOO_LARGE;
      dpk::AlignArgs A{};
      A.n = p->last_n; A.a_cat = p->last_a; A.b_cat = p->last_b; A.a_off = p->last_aoff; A.b_off = p->last_boff;
      A.max_la = p->last_max_la > 0 ? p->last_max_la : 1; A.max_lb = p->last_max_lb > 0 ? p->last_max_lb : 1;
      A.sigma = p->d_sigma; A.asz = p->asz; A.local = true;
      A.gap_open = p->gap_open; A.gap_ext = p->gap_ext;
      A.scores = p->last_scores;
      A.dirs = static_cast<uint32_t*>(p->tb_state.ptr);
      A.ends = static_cast<int32_t*>(p->tb_aux.ptr);
      if (p->affine16) {
        A.dir_stride = dpk::affine16_dir_words(A.max_la, A.max_lb);
        e = dpk::affine16_traceback(A, first, count, out, stride, out_len, coords, s, &p->launches);
      } else {
        A.dir_stride = dpk::align_affine_dir_words(A.max_la, A.max_lb);
        e = dpk::align_affine_traceback(A, first, count, out, stride, out_len, coords, s, &p->launches);
      }
      break;
    }
    case DP_NUSSINOV: {
      if (stride < p->last_max_la) return DP_E_TOO_LARGE;
      const int64_t ds = p->last_max_la > 0 ? p->last_max_la : 1;
      e = dpk::nuss_copy_db(static_cast<uint8_t*>(p->tb_state.ptr), ds, static_cast<int32_t*>(p->tb_aux.ptr), first,
                            count, out, stride, out_len, s, &p->launches);
      break;
    }
    case DP_HMM_VITERBI: {
      if (stride < p->last_max_la) return DP_E_TOO_LARGE;
      dpk::HmmArgs H{};
      H.n = p->last_n; H.x_cat = p->last_a; H.x_off = p->last_aoff; H.max_len = p->last_max_la; H.S = p->S;
      H.K = p->K; H.bp = static_cast<uint8_t*>(p->tb_state.ptr); H.final_state = static_cast<int32_t*>(p->tb_aux.ptr);
      if (p->vit_walked) H.path = static_cast<uint8_t*>(p->tb_aux2.ptr);
      e = dpk::hmm_viterbi_traceback(H, first, count, out, stride, out_len, s, &p->launches);
      break;
    }
  }
  return cuda_status(e);
}

dp_status dp_solve_batch_host(dp_plan_t p, int64_t n, const uint8_t* a_cat, const int64_t* a_off,
                              const uint8_t* b_cat, const int64_t* b_off, void* scores_out, uint8_t* tb_out,
                              int64_t tb_stride, int32_t* tb_len, int32_t* tb_coords, void* stream) {
  NvtxRange nvtx("dp_solve_batch_host");
  if (!p || n < 0 || (n > 0 && (!a_off || !a_cat || !scores_out))) return DP_E_INVALID;
  const bool align =
      p->kind == DP_EDIT || p->kind == DP_SW_LINEAR || p->kind == DP_SW_AFFINE || p->kind == DP_DIAG_LCS;
  if (align && n > 0 && (!b_off || !b_cat)) return DP_E_INVALID;
  cudaStream_t s = reinterpret_cast<cudaStream_t>(stream);
  int64_t max_la = 0, max_lb = 0;
  for (int64_t q = 0; q < n; ++q) {
    const int64_t la = a_off[q + 1] - a_off[q];
    if (la < 0) return DP_E_INVALID;
    if (la > max_la) max_la = la;
    if (align) {
      const int64_t lb = b_off[q + 1] - b_off[q];
      if (lb < 0) return DP_E_INVALID;
      if (lb > max_lb) max_lb = lb;
    }
  }
  if (max_la > p->max_la || (align && max_lb > p->max_lb)) return DP_E_TOO_LARGE;
  const int64_t abytes = n > 0 ? a_off[n] - a_off[0] : 0;
  const int64_t bbytes = (align && n > 0) ? b_off[n] - b_off[0] : 0;
  const bool tb = p->want_tb && tb_out && tb_len && p->kind != DP_HMM_FORWARD && n > 0;
  if (tb) {  // the traceback's stride requirement, checked before anything is enqueued
    const int64_t need = (p->kind == DP_NUSSINOV || p->kind == DP_HMM_VITERBI) ? max_la : max_la + max_lb;
    if (tb_stride < need) return DP_E_TOO_LARGE;
  }
  DeviceGuard guard(p->device);
  cudaError_t e = p->h_a.ensure((size_t)abytes + 16);
  if (e == cudaSuccess) e = p->h_aoff.ensure((size_t)(n + 1) * 8);
  if (e == cudaSuccess && align) e = p->h_b.ensure((size_t)bbytes + 16);
  if (e == cudaSuccess && align) e = p->h_boff.ensure((size_t)(n + 1) * 8);
  if (e == cudaSuccess) e = p->h_scores.ensure((size_t)n * 4 + 16);
  if (e == cudaSuccess && tb) e = p->h_tb.ensure((size_t)(n * tb_stride) + 16);
  if (e == cudaSuccess && tb) e = p->h_tblen.ensure((size_t)n * 4 + 16);
  if (e == cudaSuccess && tb && tb_coords) e = p->h_coords.ensure((size_t)n * 16 + 16);
  if (e == cudaSuccess && !p->s_h2d) e = cudaStreamCreateWithFlags(&p->s_h2d, cudaStreamNonBlocking);
  if (e == cudaSuccess && !p->s_d2h) e = cudaStreamCreateWithFlags(&p->s_d2h, cudaStreamNonBlocking);
  if (e == cudaSuccess && !p->ev_start) e = cudaEventCreateWithFlags(&p->ev_start, cudaEventDisableTiming);
  for (int k = 0; e == cudaSuccess && k < dp_plan::kMaxChunks; ++k) {
    if (!p->ev_in[k]) e = cudaEventCreateWithFlags(&p->ev_in[k], cudaEventDisableTiming);
    if (e == cudaSuccess && !p->ev_out[k]) e = cudaEventCreateWithFlags(&p->ev_out[k], cudaEventDisableTiming);
  }
  if (e != cudaSuccess) return cuda_status(e);
  if (n == 0) return dp_solve_batch(p, 0, nullptr, nullptr, nullptr, nullptr, 0, 0, p->h_scores.ptr, stream);
  // Chunks of the batch: chunk c is copied in on s_h2d, solved (and traced) on
  // the caller's stream, copied out on s_d2h, so the transfers of one chunk
  // overlap the solve of its neighbours. Device copies keep the host layout:
  // byte q of a_cat lives at h_a + (q - a_off[0]), so the kernels take the
  // caller's (absolute) offsets with a rebased base pointer.
  // a chunk must still fill the GPU: ~3 waves of the sweep kernels
  // (config 2, round 1: 1 / 2 / 3 / 4 / 8 / 12 chunks -> 4.53 / 3.73 / 3.55 / 3.46 / 4.14 / 4.31 ms)
  const int64_t min_chunk = align ? 16384 : (p->kind == DP_NUSSINOV ? 65536 : 32768);
  // packed SW alternates two compute streams (a chunk's sweep under the previous chunk's
  // traceback) and gains from finer chunks (config 2, 2 / 4 / 6 chunks: 3.90 / 3.22 / 3.00 ms);
  // the one-stream kinds measured best at 4 (affine SW 9.57 vs 9.95 ms at 6, short pairs 5.25 vs
  // 5.59); env DP_HOST_CHUNKS: diagnostic
  const int max_ch = p->env.host_chunks > 0 ? p->env.host_chunks : (p->kind == DP_SW_LINEAR && p->packed16 ? 6 : 4);
  int nch = (int)std::min<int64_t>(max_ch, (n + min_chunk - 1) / min_chunk);
  if (nch < 1) nch = 1;
  // chunk boundaries: the first chunk's H2D and the last chunk's D2H are exposed (nothing to
  // overlap them with), so with 3+ chunks those two are `edge` times the size of the others
  int64_t bound[dp_plan::kMaxChunks + 1];
  {
    const double edge = nch >= 3 ? p->env.host_edge : 1.0;
    const double unit = (double)n / (nch >= 3 ? 2.0 * edge + (nch - 2) : (double)nch);
    double acc = 0.0;
    bound[0] = 0;
    for (int c = 1; c < nch; ++c) {
      acc += (nch >= 3 && c == 1) ? edge : 1.0;
      bound[c] = std::min<int64_t>(n, ((int64_t)(acc * unit + 0.5) + 1) & ~int64_t(1));  // even: whole packed groups
    }
    bound[nch] = n;
  }
  uint8_t* da = static_cast<uint8_t*>(p->h_a.ptr);
  uint8_t* db = align ? static_cast<uint8_t*>(p->h_b.ptr) : nullptr;
  int64_t* dao = static_cast<int64_t*>(p->h_aoff.ptr);
  int64_t* dbo = align ? static_cast<int64_t*>(p->h_boff.ptr) : nullptr;
  // Once anything is enqueued an error path must not return while copies into or out of the
  // caller's host buffers may still run: drain every stream first (the call is synchronous).
  const bool two_cmp = p->kind == DP_SW_LINEAR && p->packed16;
  auto drain = [&](dp_status st) {
    cudaStreamSynchronize(p->s_h2d);
    cudaStreamSynchronize(s);
    if (two_cmp && p->s_cmp) cudaStreamSynchronize(p->s_cmp);
    cudaStreamSynchronize(p->s_d2h);
    return st;
  };
  e = cudaEventRecord(p->ev_start, s);  // buffers are free once earlier work on the caller's stream is done
  if (e == cudaSuccess) e = cudaStreamWaitEvent(p->s_h2d, p->ev_start, 0);
  if (e == cudaSuccess) e = cudaMemcpyAsync(dao, a_off, (n + 1) * 8, cudaMemcpyHostToDevice, p->s_h2d);
  if (e == cudaSuccess && align) e = cudaMemcpyAsync(dbo, b_off, (n + 1) * 8, cudaMemcpyHostToDevice, p->s_h2d);
  if (e != cudaSuccess) return drain(cuda_status(e));
  // Packed SW keeps all of a solve's retained state in tb_state, so consecutive chunks can
  // alternate between two compute streams and two state buffers: chunk c+1's sweep then fills the
  // SMs while chunk c's traceback drains (other kinds stay on the caller's stream).
  const bool two = p->kind == DP_SW_LINEAR && p->packed16 && nch > 1;
  if (two && !p->s_cmp) {
    e = cudaStreamCreateWithFlags(&p->s_cmp, cudaStreamNonBlocking);
    if (e == cudaSuccess) e = cudaStreamWaitEvent(p->s_cmp, p->ev_start, 0);
    if (e != cudaSuccess) return drain(cuda_status(e));
  } else if (two) {
    e = cudaStreamWaitEvent(p->s_cmp, p->ev_start, 0);
    if (e != cudaSuccess) return drain(cuda_status(e));
  }
  int installed = 0;  // which state buffer is in p->tb_state
  for (int c = 0; c < nch; ++c) {
    const int64_t k0 = bound[c], k1 = std::max(k0, bound[c + 1]), nk = k1 - k0;
    if (nk <= 0) continue;
    const cudaStream_t sc = (two && (c & 1)) ? p->s_cmp : s;
    void* const scv = reinterpret_cast<void*>(sc);
    if (two && (c & 1) != installed) {
      std::swap(p->tb_state, p->tb_state_alt);
      installed = c & 1;
    }
    e = cudaMemcpyAsync(da + (a_off[k0] - a_off[0]), a_cat + a_off[k0], a_off[k1] - a_off[k0],
                        cudaMemcpyHostToDevice, p->s_h2d);
    if (e == cudaSuccess && align)
      e = cudaMemcpyAsync(db + (b_off[k0] - b_off[0]), b_cat + b_off[k0], b_off[k1] - b_off[k0],
                          cudaMemcpyHostToDevice, p->s_h2d);
    if (e == cudaSuccess) e = cudaEventRecord(p->ev_in[c], p->s_h2d);
    if (e == cudaSuccess) e = cudaStreamWaitEvent(sc, p->ev_in[c], 0);
    if (e != cudaSuccess) return drain(cuda_status(e));
    int32_t* dsc = static_cast<int32_t*>(p->h_scores.ptr) + k0;
    dp_status st = dp_solve_batch(p, nk, da - a_off[0], dao + k0, align ? db - b_off[0] : nullptr,
                                  align ? dbo + k0 : nullptr, max_la, max_lb, dsc, scv);
    if (st != DP_OK) return drain(st);
    uint8_t* dtb = tb ? static_cast<uint8_t*>(p->h_tb.ptr) + k0 * tb_stride : nullptr;
    int32_t* dtl = tb ? static_cast<int32_t*>(p->h_tblen.ptr) + k0 : nullptr;
    int32_t* dco = (tb && tb_coords) ? static_cast<int32_t*>(p->h_coords.ptr) + 4 * k0 : nullptr;
    if (tb) {
      st = dp_traceback(p, 0, nk, dtb, tb_stride, dtl, dco, scv);
      if (st != DP_OK) return drain(st);
    }
    e = cudaEventRecord(p->ev_out[c], sc);
    if (e == cudaSuccess) e = cudaStreamWaitEvent(p->s_d2h, p->ev_out[c], 0);
    if (e == cudaSuccess)
      e = cudaMemcpyAsync(static_cast<uint8_t*>(scores_out) + 4 * k0, dsc, nk * 4, cudaMemcpyDeviceToHost, p->s_d2h);
    if (e == cudaSuccess && tb) e = cudaMemcpyAsync(tb_out + k0 * tb_stride, dtb, nk * tb_stride,
                                                    cudaMemcpyDeviceToHost, p->s_d2h);
    if (e == cudaSuccess && tb) e = cudaMemcpyAsync(tb_len + k0, dtl, nk * 4, cudaMemcpyDeviceToHost, p->s_d2h);
    if (e == cudaSuccess && dco) e = cudaMemcpyAsync(tb_coords + 4 * k0, dco, nk * 16, cudaMemcpyDeviceToHost, p->s_d2h);
    if (e != cudaSuccess) return drain(cuda_status(e));
  }
  e = cudaStreamSynchronize(p->s_d2h);
  if (e == cudaSuccess) e = cudaStreamSynchronize(s);
  if (e == cudaSuccess && two) e = cudaStreamSynchronize(p->s_cmp);
  return cuda_status(e);
}

}  // extern "C"
