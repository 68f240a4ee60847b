/*
 * czc_oracle.c — CPU ORACLE (test infrastructure only; see czc_oracle.h for the contract).
 *
 * Plain definitions, no blocking, fusion or running sums.  Per-element arithmetic in double,
 * every sum in long double, moments two-pass centred.  Build:  gcc -O2 -fopenmp
 * -ffp-contract=off (no FMA contraction, IEEE round-to-nearest; reading R21).  OpenMP only
 * splits independent rows / window planes; their long-double partials are combined in index
 * order, so the result does not depend on the thread count beyond long-double rounding.
 */
#include "czc_oracle.h"

#include <float.h>
#include <math.h>
#include <stdlib.h>
#include <string.h>
#ifdef _OPENMP
#include <omp.h>
#endif

typedef long double ld;

int czco_threads(void) {
#ifdef _OPENMP
  return omp_get_max_threads();
#else
  return 1;
#endif
}

/* Shapes: ndim 1..4 (4-D is NEXT row f3), right-aligned into NA = 4 axes with leading 1s (an
 * axis of extent 1 is inactive).  Returns 0 if invalid. */
#define NA 4
#define CZCO_P1_CHUNK 65536   /* P1: fixed element chunks, combined in chunk order */
static int shape4(int ndim, const int64_t* dims, int64_t n[NA]) {
  if (ndim < 1 || ndim > NA || !dims) return 0;
  for (int a = 0; a < NA; a++) n[a] = 1;
  for (int i = 0; i < ndim; i++) {
    if (dims[i] < 1) return 0;
    n[NA - ndim + i] = dims[i];
  }
  return 1;
}
static void strides4(const int64_t n[NA], int64_t st[NA]) {
  st[NA - 1] = 1;
  for (int a = NA - 2; a >= 0; a--) st[a] = st[a + 1] * n[a + 1];
}
/* Per-axis window extents / steps / origins right-aligned like the shape (leading `fill`). */
static int window4(int ndim, const int64_t* v, int64_t out[NA], int64_t fill) {
  for (int a = 0; a < NA; a++) out[a] = fill;
  for (int i = 0; i < ndim; i++) out[NA - ndim + i] = v[i];
  return 1;
}

/* PDF bin rule (reading R24): floor((v - lo) / w), top edge clamped, w == 0 -> bin 0. */
static int pdf_bin(double v, double lo, double w, int nbins) {
  if (!(w > 0) || isinf(w)) return 0;
  const double q = (v - lo) / w;              /* IEEE quotient, no contraction (R21) */
  int b = (int)floor(q);
  if (b >= nbins) b = nbins - 1;
  if (b < 0) b = 0;
  return b;
}

/* The pattern definitions (czc_oracle_t.inc), once per element type: float32 inputs (the paper's
 * precision, L330) and float64 inputs (NEXT row f3).  Every sample is read as a double, so both
 * instances evaluate the same expressions. */
#define CZCO_CAT_(a, b) a##b
#define CZCO_CAT(a, b) CZCO_CAT_(a, b)
#define FN(name) CZCO_CAT(name, CZCO_SFX)

#define ELEM float
#define CZCO_SFX
#include "czc_oracle_t.inc"
#undef ELEM
#undef CZCO_SFX

#define ELEM double
#define CZCO_SFX _f64
#include "czc_oracle_t.inc"
#undef ELEM
#undef CZCO_SFX
