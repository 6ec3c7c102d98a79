// NEXT-4 consumer: occu-packing (P390-P392; R38).  First-fit bin packing of jobs by
// their predicted GPU occupancy: job j (submission order) goes to the lowest-numbered GPU
// slot whose cumulative occupancy stays <= capacity after adding it, else a new slot opens.
//
// O(n log n): a segment tree over slots keeps the minimum load of each subtree; the query
// descends to the leftmost slot whose load satisfies load + occ <= capacity.  Because
// x -> x + occ is monotone in floating point, a subtree contains a fitting slot iff its
// minimum load fits, so the descent takes exactly the slot a linear first-fit scan would —
// with the same float64 predicate and the same per-slot summation order as the oracle.
#include <math.h>
#include <stdint.h>

#include <string>
#include <vector>

#include "occu_internal.h"

extern "C" occu_status occu_pack_jobs(const float *occ, int32_t num_jobs, double capacity,
                                      int32_t *slot_of_job, double *slot_load,
                                      int32_t *num_slots) {
  if (!occ || !slot_of_job || !num_slots || num_jobs < 0) {
    occu::set_global_error("occu_pack_jobs: NULL argument or num_jobs < 0");
    return OCCU_EINVAL;
  }
  if (!(capacity > 0.0) || !isfinite(capacity)) {
    occu::set_global_error("occu_pack_jobs: capacity must be finite and > 0");
    return OCCU_EINVAL;
  }
  for (int32_t j = 0; j < num_jobs; ++j)
    if (!isfinite(occ[j])) {
      occu::set_global_error("occu_pack_jobs: non-finite predicted occupancy");
      return OCCU_EINVAL;
    }
  int size = 1;
  while (size < num_jobs) size <<= 1;
  // tree[1] is the root; leaves size..2*size-1 are slots; unopened slots hold +inf (never fit)
  std::vector<double> tree(2 * size, INFINITY), load(num_jobs > 0 ? num_jobs : 1, 0.0);
  int opened = 0;
  for (int32_t j = 0; j < num_jobs; ++j) {
    const double o = occ[j] > 0.f ? double(occ[j]) : 0.0;
    int b;
    if (opened > 0 && tree[1] + o <= capacity) {
      int v = 1;
      while (v < size) v = (tree[2 * v] + o <= capacity) ? 2 * v : 2 * v + 1;
      b = v - size;
      load[b] += o;
    } else {
      b = opened++;
      load[b] = o;
    }
    slot_of_job[j] = b;
    int v = b + size;
    tree[v] = load[b];
    for (v >>= 1; v >= 1; v >>= 1) tree[v] = fmin(tree[2 * v], tree[2 * v + 1]);
  }
  *num_slots = opened;
  if (slot_load)
    for (int b = 0; b < opened; ++b) slot_load[b] = load[b];
  return OCCU_OK;
}
