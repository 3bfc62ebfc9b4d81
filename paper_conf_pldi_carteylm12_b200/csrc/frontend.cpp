// Host front-end: dependency families -> validity criteria -> minimal-partition
// schedule (§4.4–§4.8; SURVEY.md §8(a) A1–A4).
//
// Unlike the brute-force test oracle (oracle/schedule.py, which walks every
// edge of a concrete call graph), this works symbolically on the families of
// call sites: one criterion per uniform family and two per ranged family.
#include <cstdint>
#include <cstdlib>
#include <climits>
#include <algorithm>
#include <vector>
#include <array>

#include "dp.h"

namespace {

// eq.(3) specialised to descents x_r = x + c (§4.5):
//   S(x) - S(x_r) = -a.c > 0.
// A ranged family x_r = x + c + delta e_k, delta in [lo, hi], is linear in delta,
// so the criterion holds for every delta iff it holds at both endpoints.
int64_t neg_dot(int ndim, const int32_t* a, const int32_t* off, int axis, int64_t delta) {
  int64_t s = 0;
  for (int i = 0; i < ndim; ++i) {
    int64_t c = off[i] + (i == axis ? delta : 0);
    s -= (int64_t)a[i] * c;
  }
  return s;
}

bool satisfies(int ndim, const int32_t* a, int ndeps, const dp_dep* deps) {
  for (int d = 0; d < ndeps; ++d) {
    const dp_dep& f = deps[d];
    if (f.ranged_axis < 0) {
      if (neg_dot(ndim, a, f.offset, -1, 0) <= 0) return false;
    } else {
      if (neg_dot(ndim, a, f.offset, f.ranged_axis, f.lo) <= 0) return false;
      if (neg_dot(ndim, a, f.offset, f.ranged_axis, f.hi) <= 0) return false;
    }
  }
  return true;
}

// eq.(4) linearised per sign (§4.6): the max of a_i x_i over
// 0 <= x_i < n_i sits at x_i = n_i - 1 when a_i > 0 and at 0 otherwise.
int64_t box_goal(int ndim, const int32_t* a, const int64_t* ext) {
  int64_t g = 0;
  for (int i = 0; i < ndim; ++i) g += (int64_t)std::llabs(a[i]) * (ext[i] - 1);
  return g;
}

void exact_range(int ndim, const int32_t* a, const int64_t* ext, int triangular, int64_t* lo, int64_t* hi) {
  if (triangular && ndim == 2) {
    // domain {0 <= x0 <= x1 < n}: a linear function peaks at a vertex
    int64_t n = ext[0] - 1;
    int64_t v[3] = {0, (int64_t)a[1] * n, ((int64_t)a[0] + a[1]) * n};
    *lo = v[0]; *hi = v[0];
    for (int k = 1; k < 3; ++k) { if (v[k] < *lo) *lo = v[k]; if (v[k] > *hi) *hi = v[k]; }
    return;
  }
  int64_t l = 0, h = 0;
  for (int i = 0; i < ndim; ++i) {
    int64_t t = (int64_t)a[i] * (ext[i] - 1);
    if (t < 0) l += t; else h += t;
  }
  *lo = l; *hi = h;
}

// §4.8: the window is the largest partition distance a call reaches back.
// For a ranged family whose distance depends on delta (a[axis] != 0) it is
// not known statically (the paper's "affine" case): -1.
int32_t window_of(int ndim, const int32_t* a, int ndeps, const dp_dep* deps) {
  int64_t w = 0;
  for (int d = 0; d < ndeps; ++d) {
    const dp_dep& f = deps[d];
    if (f.ranged_axis >= 0) {
      if (a[f.ranged_axis] != 0) return -1;
      int64_t v = neg_dot(ndim, a, f.offset, f.ranged_axis, f.lo);
      if (v > w) w = v;
    } else {
      int64_t v = neg_dot(ndim, a, f.offset, -1, 0);
      if (v > w) w = v;
    }
  }
  return (int32_t)w;
}

}  // namespace

extern "C" dp_status dp_schedule_derive(int ndim, const int64_t extent[], int triangular, int ndeps,
                                        const dp_dep deps[], int coeff_bound, const int32_t* user_coeff,
                                        int32_t coeff_out[], int64_t* p_lo, int64_t* p_hi, int32_t* window) {
  if (ndim < 1 || ndim > DP_MAX_DIM || !extent || ndeps < 0 || (ndeps > 0 && !deps) || !coeff_out) return DP_E_INVALID;
  if (triangular && ndim != 2) return DP_E_INVALID;
  for (int i = 0; i < ndim; ++i)
    if (extent[i] < 1) return DP_E_INVALID;
  for (int d = 0; d < ndeps; ++d)
    if (deps[d].ranged_axis >= ndim || (deps[d].ranged_axis >= 0 && deps[d].lo > deps[d].hi)) return DP_E_INVALID;
  int B = coeff_bound > 0 ? coeff_bound : 10;  // L403–L404

  int32_t best[DP_MAX_DIM] = {0, 0, 0, 0};
  bool found = false;
  if (user_coeff) {  // verify a user-given schedule (L326, L345–L348)
    for (int i = 0; i < ndim; ++i) best[i] = user_coeff[i];
    found = satisfies(ndim, best, ndeps, deps);
  } else {
    // lexicographic enumeration of [-B, B]^ndim; strict '<' keeps the first minimum
    int32_t a[DP_MAX_DIM];
    for (int i = 0; i < ndim; ++i) a[i] = -B;
    int64_t best_goal = INT64_MAX;
    for (;;) {
      if (satisfies(ndim, a, ndeps, deps)) {
        int64_t g = box_goal(ndim, a, extent);
        if (g < best_goal) {
          best_goal = g;
          for (int i = 0; i < ndim; ++i) best[i] = a[i];
          found = true;
        }
      }
      int k = ndim - 1;
      while (k >= 0 && a[k] == B) { a[k] = -B; --k; }
      if (k < 0) break;
      ++a[k];
    }
  }
  if (!found) return DP_E_NO_SCHEDULE;
  for (int i = 0; i < ndim; ++i) coeff_out[i] = best[i];
  int64_t lo, hi;
  exact_range(ndim, best, extent, triangular, &lo, &hi);
  if (p_lo) *p_lo = lo;
  if (p_hi) *p_hi = hi;
  if (window) *window = window_of(ndim, best, ndeps, deps);
  return DP_OK;
}

/*
 * §4.7 conditional parallelisation (L379–L402). For each order pi of the
 * dimensions (ndim! of them, identity first, std::next_permutation order) the
 * valid a in [-B, B]^ndim minimising |a_pi1|, then |a_pi2|, ... (each
 * dimension minimised in turn with the constraints of the earlier ones
 * propagated; R-SCHED-COND); among the valid a with that tuple of
 * magnitudes the lexicographically smallest. Distinct results are candidates,
 * each minimal for some extents vector; dp_schedule_select picks one per problem.
 */
extern "C" dp_status dp_schedule_conditional(int ndim, int ndeps, const dp_dep deps[], int coeff_bound, int max_out,
                                             int32_t coeffs_out[], int* count) {
  if (ndim < 1 || ndim > DP_MAX_DIM || ndeps < 0 || (ndeps > 0 && !deps) || max_out < 1 || !coeffs_out || !count)
    return DP_E_INVALID;
  for (int d = 0; d < ndeps; ++d)
    if (deps[d].ranged_axis >= ndim || (deps[d].ranged_axis >= 0 && deps[d].lo > deps[d].hi)) return DP_E_INVALID;
  const int B = coeff_bound > 0 ? coeff_bound : 10;
  // the valid coefficient vectors (eq.3 per family)
  std::vector<std::array<int32_t, DP_MAX_DIM>> valid;
  {
    std::array<int32_t, DP_MAX_DIM> a{};
    for (int i = 0; i < ndim; ++i) a[i] = -B;
    for (;;) {
      if (satisfies(ndim, a.data(), ndeps, deps)) valid.push_back(a);
      int k = ndim - 1;
      while (k >= 0 && a[k] == B) { a[k] = -B; --k; }
      if (k < 0) break;
      ++a[k];
    }
  }
  *count = 0;
  if (valid.empty()) return DP_E_NO_SCHEDULE;
  int perm[DP_MAX_DIM];
  for (int i = 0; i < ndim; ++i) perm[i] = i;
  do {
    // minimise |a_perm[k]| in turn, keeping only the vectors that attain each minimum
    std::vector<const std::array<int32_t, DP_MAX_DIM>*> cand;
    for (const auto& a : valid) cand.push_back(&a);
    for (int k = 0; k < ndim; ++k) {
      int32_t m = INT32_MAX;
      for (const auto* a : cand) m = std::min(m, std::abs((*a)[perm[k]]));
      std::vector<const std::array<int32_t, DP_MAX_DIM>*> keep;
      for (const auto* a : cand)
        if (std::abs((*a)[perm[k]]) == m) keep.push_back(a);
      cand.swap(keep);
    }
    // sign ties: the lexicographically smallest (valid is in lexicographic order)
    const auto& best = *cand.front();
    bool dup = false;
    for (int c = 0; c < *count && !dup; ++c)
      dup = std::equal(best.begin(), best.begin() + ndim, coeffs_out + (size_t)c * ndim);
    if (!dup) {
      if (*count == max_out) return DP_E_TOO_LARGE;
      std::copy(best.begin(), best.begin() + ndim, coeffs_out + (size_t)(*count) * ndim);
      ++*count;
    }
  } while (std::next_permutation(perm, perm + ndim));
  return DP_OK;
}

/* Run-time half of §4.7 (L384–L386): the candidate with the smallest box range
 * sum |a_i| (extent_i - 1) for this problem (eq.4); the first on ties. */
extern "C" int dp_schedule_select(int ndim, int count, const int32_t coeffs[], const int64_t extent[]) {
  if (ndim < 1 || ndim > DP_MAX_DIM || count < 1 || !coeffs || !extent) return -1;
  int best = 0;
  int64_t bg = INT64_MAX;
  for (int c = 0; c < count; ++c) {
    const int64_t g = box_goal(ndim, coeffs + (size_t)c * ndim, extent);
    if (g < bg) { bg = g; best = c; }
  }
  return best;
}
