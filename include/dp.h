/*
 * dp.h — C ABI of the B200 hyperplane DP library (libdp.so).
 *
 * The library evaluates a recursion-equation dynamic-programming table
 * partition by partition ("hyperplane"/wavefront), the partitions being those
 * of the affine schedule S_f = a1 x1 + ... + an xn that the paper's static
 * dependency analysis derives (Cartey, Lyngsø & de Moor, PLDI 2012; citations
 * `Lnnn` are lines of PAPER.md's decoded fulltext):
 *   - the user states a recursion over the indices of calling parameters
 *     (sequences, a substitution matrix, an HMM), §3.1–§3.2;
 *   - the framework tabulates it bottom-up and returns the top call (L93–L96);
 *   - `map` applies it to many argument sets (L194–L195)  -> dp_solve_batch;
 *   - a user-given schedule is verified (L326, L345–L348) -> dp_desc.user_coeff.
 *
 * Ownership: the caller owns every input/output buffer; the library never
 * frees caller memory. A plan owns its device workspace and the state retained
 * for dp_traceback until the next solve or dp_plan_destroy. A plan is not
 * thread-safe; distinct plans are independent.
 *
 * Errors: argument errors return synchronously with nothing enqueued. Launch
 * errors return DP_E_CUDA; asynchronous faults surface at stream sync. No
 * exception or abort crosses the ABI.
 *
 * Alphabet codes >= alphabet_size are a caller error (undefined in the kernel;
 * the Python binding checks them in debug mode).
 */
#ifndef DP_H_
#define DP_H_

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define DP_ABI_VERSION 4
#define DP_MAX_DIM 4

typedef enum dp_status {
  DP_OK = 0,
  DP_E_INVALID = 1,      /* bad argument (null pointer, negative size, bad kind ...) */
  DP_E_NO_SCHEDULE = 2,  /* the validity criteria (eq.3) are infeasible: cyclic dependencies */
  DP_E_UNSUPPORTED = 3,  /* valid request this build does not implement (e.g. forward traceback) */
  DP_E_TOO_LARGE = 4,    /* a length exceeds the plan maximum or a device limit */
  DP_E_NOMEM = 5,        /* device or host allocation failed */
  DP_E_CUDA = 6,         /* a CUDA call failed */
  DP_E_NO_TRACEBACK = 7  /* dp_traceback without want_traceback or before a solve */
} dp_status;

/* The paper's case-study recurrences (SURVEY.md §8(a) A6a–A6d). */
typedef enum dp_kind {
  DP_EDIT = 0,        /* Fig.7, edit distance d(|s|,|t|), int32 */
  DP_SW_LINEAR = 1,   /* §6.1 L502–L507 + §5.1: local alignment, linear gap, int32 score */
  DP_NUSSINOV = 2,    /* interval DP with max over split k (ref [3], L598), int32 #pairs */
  DP_HMM_FORWARD = 3, /* Fig.11a, natural-log likelihood, float32 */
  DP_HMM_VITERBI = 4, /* max-variant of Fig.11a (L463–L464), int32 milli-bit score */
  DP_SW_AFFINE = 5    /* SURVEY §8(f) NEXT 1 (Gotoh, L509–L520; mutual recursion = Further Work L585–L589):
                         local alignment, gap of length k costs gap_open + k * gap_extend, int32 score */,
  DP_DIAG_LCS = 6,    /* the §4.7 example f(x,y) = ... f(x-1,y-1) ... (L386–L388) as the
                         longest common substring, int32; its schedule is chosen per problem among the
                         conditional candidates (S = i when |a| < |b|, else S = j); no traceback (ABI 3) */
  DP_PROFILE_FORWARD = 7 /* profile-HMM forward (§6.3; Durbin ch.5, ref [3]):
                         one profile of n_positions match positions against each sequence a, natural-log
                         likelihood, float32; three tables (M, I, D) over (position, index), schedule (1,1);
                         no traceback (ABI 4) */
} dp_kind;

/*
 * One dependency family of a recurrence (§4.4–§4.5): each recursive call site
 * f(x_r) with a uniform descent x_r = x + offset, or ranged along one axis:
 * x_r = x + offset + delta * e_{ranged_axis}, delta in [lo, hi] (a loop
 * variable with runtime range, §5; e.g. Nussinov's split k).
 */
typedef struct dp_dep {
  int32_t offset[DP_MAX_DIM];
  int32_t ranged_axis; /* -1 = uniform */
  int64_t lo, hi;      /* inclusive delta range when ranged */
} dp_dep;

/*
 * dp_schedule_derive — the host front-end (SURVEY.md §8(a) A1–A4), pure CPU.
 * Finds integer a in [-coeff_bound, coeff_bound]^ndim (coeff_bound <= 0 -> 10,
 * L403–L404) satisfying the validity criteria -a.c > 0 for every uniform
 * family and for both delta endpoints of every ranged family (eq.3),
 * minimising the box range sum_i |a_i| (extent_i - 1) (eq.4); ties
 * go to the lexicographically smallest a (DESIGN.md R-SCHED-TIE).
 * Outputs: coeff_out[ndim]; [*p_lo, *p_hi] = exact partition range over the
 * domain (the box, or the triangle x0 <= x1 when triangular != 0, ndim == 2);
 * *window = max over uniform families of -a.c (§4.8), or -1 when any family is
 * ranged (no sliding window). Returns DP_E_NO_SCHEDULE when infeasible.
 * If user_coeff != NULL the function instead VERIFIES that schedule against
 * the same criteria (L326) and fills the outputs for it, or returns
 * DP_E_NO_SCHEDULE if it is invalid.
 */
dp_status dp_schedule_derive(int ndim, const int64_t extent[], int triangular, int ndeps, const dp_dep deps[],
                             int coeff_bound, const int32_t* user_coeff, int32_t coeff_out[], int64_t* p_lo,
                             int64_t* p_hi, int32_t* window);

/*
 * dp_schedule_conditional — §4.7 conditional parallelisation (L379–L402), pure
 * CPU. "Different problem sizes may therefore require different schedules"
 * (L380–L381): for each of the ndim! orders of the dimensions, the valid a in
 * [-coeff_bound, coeff_bound]^ndim (criteria as dp_schedule_derive) that
 * minimises |a| dimension by dimension in that order (L398–L401; magnitudes per
 * DESIGN.md R-SCHED-COND), sign ties to the lexicographically smallest a.
 * Distinct results (each minimal for some extents) go to coeffs_out as
 * count x ndim int32, identity order first. max_out bounds the output
 * (DP_E_TOO_LARGE if exceeded; ndim! <= 24 always suffices).
 * Returns DP_E_NO_SCHEDULE (count 0) when no valid a exists, DP_E_INVALID on
 * bad arguments. Example (L386–L388): f(x-1, y-1) -> {(0,1), (1,0)}.
 */
dp_status dp_schedule_conditional(int ndim, int ndeps, const dp_dep deps[], int coeff_bound, int max_out,
                                  int32_t coeffs_out[], int* count);

/*
 * dp_schedule_select — the run-time half of §4.7 (L384–L386): index of the
 * candidate (coeffs: count x ndim, from dp_schedule_conditional) with the
 * smallest box range sum_i |a_i| (extent_i - 1) (eq.4) for one problem's
 * extents; the first on ties. -1 on bad arguments.
 */
int dp_schedule_select(int ndim, int count, const int32_t coeffs[], const int64_t extent[]);

/*
 * Plan description. POD; set struct_size = sizeof(dp_desc). All pointers are
 * HOST pointers and are copied into the plan at dp_plan_create.
 */
typedef struct dp_desc {
  uint32_t struct_size;
  int32_t kind;              /* dp_kind */
  int64_t max_len_a;         /* max |a| over the batches this plan will see (rows / RNA length / T) */
  int64_t max_len_b;         /* max |b| (alignment kinds only) */
  /* alignment: substitution matrix extension (§5.1) */
  int32_t alphabet_size;     /* <= 32 for alignment kinds, 4 for Nussinov/HMM emissions */
  const int8_t* sigma;       /* [alphabet_size x alphabet_size] row = code of a, col = code of b (SW only) */
  int32_t gap;               /* linear gap penalty g > 0 (SW only; edit uses unit costs) */
  /* Nussinov */
  const uint8_t* pair_mask;  /* [4 x 4], 1 where bases may pair */
  int32_t min_hairpin;       /* h: pair (i,j) needs j - i - 1 >= h */
  /* HMM extension (§5.2): n_states <= 64, emission alphabet = alphabet_size <= 16 */
  int32_t n_states;
  const float* pi;           /* [S] start-transition probabilities (forward) */
  const float* A;            /* [S x S] A[p*S + s] = t_{p,s} (forward) */
  const float* E;            /* [S x K] E[s*K + c] = e_{s,c} (forward) */
  const int32_t* lpi;        /* [S]     milli-bit scores (Viterbi) */
  const int32_t* lA;         /* [S x S] */
  const int32_t* lE;         /* [S x K] */
  /* schedule options */
  int32_t coeff_bound;       /* 0 -> 10 */
  const int32_t* user_coeff; /* optional user schedule to verify (length = recurrence ndim) */
  int32_t want_traceback;    /* retain state for dp_traceback */
  /* affine gaps (DP_SW_AFFINE; ABI 2): gap of length k costs gap_open + k * gap_extend */
  int32_t gap_open;          /* >= 0 */
  int32_t gap_extend;        /* >= 1 */
  /* profile HMM (DP_PROFILE_FORWARD; ABI 4). Positions j = 0..L (L = n_positions >= 1); state M_0 is the
   * begin state, M_{L+1} the end state, D_0 does not exist. alphabet_size = K <= 32 emission codes. */
  int32_t n_positions;       /* L */
  const float* ptrans;       /* [(L+1) x 9]: ptrans[9 j + 3 f + t] = probability from (M_j, I_j, D_j)[f] to
                                (M_{j+1}, I_j, D_{j+1})[t]; at j = L the "to M_{L+1}" slot is the end */
  const float* pemit_m;      /* [(L+1) x K] match emissions e_{M_j}(c) (row 0 unused) */
  const float* pemit_i;      /* [(L+1) x K] insert emissions e_{I_j}(c) */
} dp_desc;

typedef struct dp_plan* dp_plan_t;

int dp_abi_version(void);
const char* dp_status_string(dp_status s);

/* Validates d, derives (or verifies) the schedule via dp_schedule_derive, picks
 * the kernel variant, copies the scoring parameters to the current CUDA device.
 * Variants: SW_LINEAR with max(max_len_a, max_len_b) <= 64 runs the
 * inter-task kernel (one pair per thread; the short side of the §6.1 hybrid), longer
 * plans the intra-task warp kernels (two problems per warp in s16x2 when the score
 * range allows, else int32). NUSSINOV picks per batch at solve time: a few problems of
 * <= 128 nt -> one small CTA each; a few (<= 64) of 129..1024 nt -> one thread-block
 * cluster each, table in distributed shared memory; one problem > 1024 nt -> the whole
 * grid (cooperative launch); otherwise one warp per problem. Results are identical
 * whichever variant runs. DP_* environment variables, read here once per plan, force
 * variants for tests and measurements only. */
dp_status dp_plan_create(const dp_desc* d, dp_plan_t* out);
void dp_plan_destroy(dp_plan_t p);

/* The schedule the plan executes (A3/A4), for tests. coeff has room for DP_MAX_DIM. */
dp_status dp_plan_get_schedule(dp_plan_t p, int32_t coeff[], int* ndim, int64_t* p_lo, int64_t* p_hi,
                               int32_t* window);

/*
 * dp_solve_batch — the `map` primitive. All pointers are DEVICE pointers:
 *   a_cat/a_off: n sequences concatenated (uint8 codes), a_off[n+1] int64;
 *   b_cat/b_off: second sequences (alignment kinds), else NULL;
 *   scores_out:  n x int32 (EDIT, SW, NUSSINOV, VITERBI) or n x float32 (HMM_FORWARD,
 *                PROFILE_FORWARD: natural-log likelihood, -inf for P = 0), in input order.
 * Asynchronous on `stream` (a cudaStream_t; NULL = legacy default stream).
 * max_len_a/max_len_b of THIS batch must be supplied (<= the plan maxima);
 * they size the launch without reading device offsets on the host.
 */
dp_status dp_solve_batch(dp_plan_t p, int64_t n, const uint8_t* a_cat, const int64_t* a_off, const uint8_t* b_cat,
                         const int64_t* b_off, int64_t max_len_a, int64_t max_len_b, void* scores_out, void* stream);

/* One problem; same as dp_solve_batch with n = 1 and device buffers. */
dp_status dp_solve(dp_plan_t p, const uint8_t* a, int64_t len_a, const uint8_t* b, int64_t len_b, void* score_out,
                   void* stream);

/*
 * dp_solve_batch_host — the same computation from HOST buffers (the paper's
 * timing convention includes H2D/D2H, L492–L494): copies inputs into plan
 * workspace, solves, copies scores back to scores_out (host), and, when the
 * plan wants tracebacks and tb_out != NULL, runs dp_traceback for the whole
 * batch into the host buffers tb_out / tb_len / tb_coords. Synchronous.
 * Host buffers should be pinned for full PCIe bandwidth.
 */
dp_status dp_solve_batch_host(dp_plan_t p, int64_t n, const uint8_t* a_cat, const int64_t* a_off,
                              const uint8_t* b_cat, const int64_t* b_off, void* scores_out, uint8_t* tb_out,
                              int64_t tb_stride, int32_t* tb_len, int32_t* tb_coords, void* stream);

/*
 * dp_traceback — canonical traceback of problems [first, first+count) of the
 * most recent solve on this plan (needs want_traceback). DEVICE outputs:
 *   out[count x stride]: EDIT/SW ops 'M' 'X' 'D' 'I' (start -> end);
 *                        NUSSINOV dot-bracket; VITERBI uint8 state ids (0..S-1);
 *   out_len[count]: bytes written per problem (int32);
 *   coords[count x 4] (optional, alignment kinds): start_i, start_j, end_i, end_j
 *   (1-based DP cell indices; the alignment covers a[start_i:end_i], b[start_j:end_j]).
 * Tie-breaks (DESIGN.md R-TB-*): alignment diagonal > up > left, SW end cell =
 * first maximum in row-major order, stop at H = 0; Nussinov Durbin order with
 * the smallest split k; Viterbi lowest final state / lowest predecessor.
 * Returns DP_E_TOO_LARGE if stride is smaller than a traceback.
 */
dp_status dp_traceback(dp_plan_t p, int64_t first, int64_t count, uint8_t* out, int64_t stride, int32_t* out_len,
                       int32_t* coords, void* stream);

/* Kernels launched by the most recent solve/traceback calls on this plan (for the
 * bench's gpu_launches accounting). */
int64_t dp_plan_launch_count(dp_plan_t p);

/* The kernel family the most recent dp_solve_batch / dp_solve / dp_solve_batch_host on this plan
 * ran (DESIGN.md §3 names: "k_sw16", "k_sw_inter", "k_align", "k_affine16", "k_align_affine", "k_diag",
 * "k_nuss_small", "k_nuss_cluster", "k_nuss_batch", "k_nuss_grid2", "k_nuss_cell",
 * "k_forward_tc", "k_forward", "k_viterbi16", "k_viterbi", "k_phmm_forward"); "" before the
 * first solve or for a NULL plan. Static storage; valid for the life of the library. Tests
 * and the bench use it to check which variant a plan's guards picked. */
const char* dp_plan_last_variant(dp_plan_t p);

#ifdef __cplusplus
}
#endif
#endif /* DP_H_ */
