// NEXT-3: the analytic wasted-GPU-time model of PAPER.md §5 (eqs. 1-8), as a
// pure C function so a scheduler can evaluate JIT vs periodic checkpointing
// with the capture / restore times this library measures on B200.
#include <math.h>

#include "jitc_internal.h"

using namespace jitc;

extern "C" jitc_status jitc_waste_model(int32_t kind, double n_gpus, double f, double o, double r, double m,
                                        double o_jit, double c, double* c_opt, double* w, double* w_f) {
  if (!w || !w_f || n_gpus <= 0 || f < 0 || o < 0 || r < 0 || m < 0 || o_jit < 0) {
    set_error("jitc_waste_model: bad argument");
    return JITC_EINVAL;
  }
  const double N = n_gpus;
  double cs = (o > 0) ? sqrt(N * f / (2.0 * o)) : 0.0;  // eq. 3 (printed "2α" read as 2o)
  double x;
  switch (kind) {
    case JITC_MODEL_PERIODIC_OPTIMAL:  // eq. 5: eq. 1 at c = c*
      x = 2.0 * sqrt(N * f * o / 2.0) + N * f * r;
      break;
    case JITC_MODEL_PERIODIC:  // eq. 1 / (N t) at the given frequency c
      if (c <= 0) {
        set_error("jitc_waste_model: periodic frequency must be > 0");
        return JITC_EINVAL;
      }
      x = c * o + N * f * r + N * f / (2.0 * c);
      break;
    case JITC_MODEL_USER_JIT:  // eq. 7 / (N t)
      x = f * o + o_jit + N * f * r + N * f * m / 2.0;
      break;
    case JITC_MODEL_TRANSPARENT_JIT:  // eq. 8 / (N t)
      x = o_jit + N * f * m / 2.0;
      break;
    default:
      set_error("jitc_waste_model: bad kind");
      return JITC_EINVAL;
  }
  if (c_opt) *c_opt = cs;
  *w = x;
  *w_f = x / (1.0 + x);  // eq. 6
  return JITC_OK;
}
