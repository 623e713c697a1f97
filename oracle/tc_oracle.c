/*
 * tc_oracle.c — CPU ORACLE for direct tensor contraction.  TEST INFRASTRUCTURE ONLY.
 * See tc_oracle.h for the definition followed (eq. (1),
 * L138/L145/L149) and for who may load this library.  Shares no code with libtc.
 *
 * Build: gcc -O3 -march=native -fopenmp -ffp-contract=off -fPIC -shared -o libtc_oracle_<host>.so
 *        tc_oracle.c -lm   (oracle/__init__.py builds one library per host CPU)
 * (-ffp-contract=off: every term is a plain multiply followed by a plain add.)
 */
#include "tc_oracle.h"

#include <ctype.h>
#include <math.h>
#include <stdlib.h>
#include <string.h>
#ifdef _OPENMP
#include <omp.h>
#endif

enum { OK = 0, E_ARG = 1, E_PARSE = 2, E_INDEX = 3, E_EXTENT = 4, E_UNSUP = 5 };
enum { MAX_RANK = 8, MAX_IDX = 16, MAX_NAME = 32 };

/* ---------------------------------------------------------------- parsed form */
typedef struct {
  int nidx;                         /* distinct index names                       */
  char name[MAX_IDX][MAX_NAME];
  long long ext[MAX_IDX];           /* extent per index                           */
  int rank[3];                      /* 0 = C, 1 = A, 2 = B                        */
  int pos[3][MAX_RANK];             /* index id at each position; pos 0 = FVI      */
  long long stride[3][MAX_IDX];     /* element stride of index id in tensor t (0 if absent) */
  long long numel[3];
} Spec;

static int find_name(const Spec *s, const char *nm) {
  for (int i = 0; i < s->nidx; i++)
    if (strcmp(s->name[i], nm) == 0) return i;
  return -1;
}

/* Adds a position to tensor t.  Returns status. */
static int add_pos(Spec *s, int t, const char *nm, int *too_many) {
  int id = find_name(s, nm);
  if (id < 0) {
    if (s->nidx >= MAX_IDX) { *too_many = 1; return OK; }
    id = s->nidx++;
    strncpy(s->name[id], nm, MAX_NAME - 1);
    s->name[id][MAX_NAME - 1] = 0;
  }
  if (s->rank[t] >= MAX_RANK) { *too_many = 1; return OK; }
  s->pos[t][s->rank[t]++] = id;
  return OK;
}

static const char *skip_ws(const char *p) { while (*p && isspace((unsigned char)*p)) p++; return p; }

/* Bracket form: NAME[i,j,...] = NAME[...] * NAME[...] */
static int parse_bracket(Spec *s, const char *e, int *too_many) {
  const char *p = skip_ws(e);
  for (int t = 0; t < 3; t++) {
    if (!(isalpha((unsigned char)*p) || *p == '_')) return E_PARSE;
    while (isalnum((unsigned char)*p) || *p == '_') p++;
    p = skip_ws(p);
    if (*p != '[') return E_PARSE;
    p = skip_ws(p + 1);
    if (*p != ']') {
      for (;;) {
        char nm[MAX_NAME]; int n = 0;
        if (!(isalpha((unsigned char)*p) || *p == '_')) return E_PARSE;
        while (isalnum((unsigned char)*p) || *p == '_') {
          if (n >= MAX_NAME - 1) return E_PARSE;
          nm[n++] = *p++;
        }
        nm[n] = 0;
        add_pos(s, t, nm, too_many);
        p = skip_ws(p);
        if (*p == ',') { p = skip_ws(p + 1); continue; }
        if (*p == ']') break;
        return E_PARSE;
      }
    }
    p = skip_ws(p + 1);
    if (t == 0) { if (*p != '=') return E_PARSE; p = skip_ws(p + 1); }
    else if (t == 1) { if (*p != '*') return E_PARSE; p = skip_ws(p + 1); }
  }
  return *p == 0 ? OK : E_PARSE;
}

/* TCCG form: "abcd-aebf-dfce" = C-A-B, one letter per index. */
static int parse_tccg(Spec *s, const char *e, int *too_many) {
  const char *p = skip_ws(e);
  for (int t = 0; t < 3; t++) {
    int n = 0;
    while (isalpha((unsigned char)*p)) {
      char nm[2] = {*p, 0};
      add_pos(s, t, nm, too_many);
      p++; n++;
    }
    if (n == 0) return E_PARSE;
    if (t < 2) { if (*p != '-') return E_PARSE; p++; }
  }
  p = skip_ws(p);
  return *p == 0 ? OK : E_PARSE;
}

/* Count occurrences of index id in tensor t. */
static int occurs(const Spec *s, int t, int id) {
  int c = 0;
  for (int k = 0; k < s->rank[t]; k++) c += s->pos[t][k] == id;
  return c;
}

static int parse_all(Spec *s, const char *expr, const char *extents) {
  memset(s, 0, sizeof(*s));
  if (!expr || !extents) return E_ARG;
  int too_many = 0, st;
  /* 1. expression syntax */
  st = strchr(expr, '[') ? parse_bracket(s, expr, &too_many) : parse_tccg(s, expr, &too_many);
  if (st) return st;
  /* 2. repeated index inside one tensor */
  if (!too_many)
    for (int t = 0; t < 3; t++)
      for (int id = 0; id < s->nidx; id++)
        if (occurs(s, t, id) > 1) return E_INDEX;
  /* 3. limits: rank <= 8 per tensor, <= 16 distinct indices */
  if (too_many) return E_UNSUP;
  /* 4. each index in exactly two of the three tensors, or in all three: a batch
        (Hadamard) index, SURVEY 8(f) NEXT-3 — C[..h..] = sum A[..h..] B[..h..] for every h,
        which the loop below already computes (h is decoded from C and read in A and B) */
  for (int id = 0; id < s->nidx; id++) {
    int c = occurs(s, 0, id) + occurs(s, 1, id) + occurs(s, 2, id);
    if (c != 2 && c != 3) return E_INDEX;
  }
  /* 5. extents syntax: "name:int;name:int" */
  char names[64][MAX_NAME]; long long vals[64]; int nent = 0;
  const char *p = extents;
  for (;;) {
    p = skip_ws(p);
    if (*p == 0) break;
    if (*p == ';') { p++; continue; }
    char nm[MAX_NAME]; int n = 0;
    if (!(isalpha((unsigned char)*p) || *p == '_')) return E_PARSE;
    while (isalnum((unsigned char)*p) || *p == '_') {
      if (n >= MAX_NAME - 1) return E_PARSE;
      nm[n++] = *p++;
    }
    nm[n] = 0;
    p = skip_ws(p);
    if (*p != ':') return E_PARSE;
    p = skip_ws(p + 1);
    int neg = 0;
    if (*p == '-' || *p == '+') { neg = *p == '-'; p++; }
    if (!isdigit((unsigned char)*p)) return E_PARSE;
    long long v = 0; int big = 0;
    while (isdigit((unsigned char)*p)) {
      if (v > 100000000000000LL) big = 1; else v = v * 10 + (*p - '0');
      p++;
    }
    if (big) v = 0x7fffffffffffffffLL;
    p = skip_ws(p);
    if (*p != ';' && *p != 0) return E_PARSE;
    if (nent >= 64) return E_PARSE;
    strcpy(names[nent], nm);
    vals[nent++] = neg ? -v : v;
  }
  /* 6. unknown / duplicated / missing index in the extents */
  int seen[MAX_IDX] = {0};
  for (int k = 0; k < nent; k++) {
    int id = find_name(s, names[k]);
    if (id < 0) return E_INDEX;
    if (seen[id]++) return E_INDEX;
    s->ext[id] = vals[k];
  }
  for (int id = 0; id < s->nidx; id++) if (!seen[id]) return E_INDEX;
  /* 7. extent values */
  for (int id = 0; id < s->nidx; id++) if (s->ext[id] < 1) return E_EXTENT;
  /* 8. element counts must fit int64: every tensor and the whole iteration space */
  long double all = 1;
  for (int id = 0; id < s->nidx; id++) all *= (long double)s->ext[id];
  if (all >= 9223372036854775808.0L) return E_EXTENT;
  /* column-major generalised strides (first listed index is the FVI) */
  for (int t = 0; t < 3; t++) {
    long long st1 = 1;
    for (int k = 0; k < s->rank[t]; k++) {
      s->stride[t][s->pos[t][k]] = st1;
      st1 *= s->ext[s->pos[t][k]];
    }
    s->numel[t] = st1;
  }
  return OK;
}

int tco_check(const char *expr, const char *extents) {
  Spec s;
  return parse_all(&s, expr, extents);
}

int64_t tco_numel(const char *expr, const char *extents, int t) {
  Spec s;
  if (t < 0 || t > 2 || parse_all(&s, expr, extents)) return -1;
  return s.numel[t];
}

int tco_max_threads(void) {
#ifdef _OPENMP
  return omp_get_max_threads();
#else
  return 1;
#endif
}

/* ---------------------------------------------------------------- element access */
static double load_elem(const void *p, int dtype, long long off) {
  switch (dtype) {
    case 0: return ((const double *)p)[off];
    case 1: case 2: return (double)((const float *)p)[off];
    default: {
      unsigned int bits = (unsigned int)((const unsigned short *)p)[off] << 16;
      float f; memcpy(&f, &bits, 4);
      return (double)f;
    }
  }
}

/* Round-to-nearest-even from double straight to bfloat16 (8 significant bits). */
static unsigned short to_bf16(double x) {
  float f;
  if (isnan(x)) { f = (float)x; }
  else if (isinf(x) || x == 0.0) { f = (float)x; }
  else {
    int e; frexp(x, &e);                 /* |x| = m * 2^e, 0.5 <= m < 1 */
    int q = e - 8;                       /* quantum of an 8-significant-bit value */
    if (q < -133) q = -133;              /* bf16 subnormal quantum (2^-126 * 2^-7) */
    double y = ldexp(nearbyint(ldexp(x, -q)), q);
    if (fabs(y) > 3.3895313892515355e38) y = copysign(INFINITY, x);
    f = (float)y;                        /* exact: y is representable in bf16 */
  }
  unsigned int bits; memcpy(&bits, &f, 4);
  if (isnan(x)) return (unsigned short)((bits >> 16) | 0x40);
  return (unsigned short)(bits >> 16);
}

static void store_elem(void *p, int dtype, long long off, double v) {
  switch (dtype) {
    case 0: ((double *)p)[off] = v; break;
    case 1: case 2: ((float *)p)[off] = (float)v; break;   /* C cast: RNE */
    default: ((unsigned short *)p)[off] = to_bf16(v); break;
  }
}

/* ---------------------------------------------------------------- the contraction */
/* C[x] for one C linear index x (C's first index fastest). */
static void one_element(const Spec *s, int dtype, const void *A, const void *B, const void *Cin,
                        double alpha, double beta, long long x, int exact, double *val, double *scale) {
  long long digit[MAX_IDX] = {0};
  /* decode x in C's mixed radix, first index fastest */
  long long r = x;
  for (int k = 0; k < s->rank[0]; k++) {
    int id = s->pos[0][k];
    digit[id] = r % s->ext[id];
    r /= s->ext[id];
  }
  /* internal indices, listed in A's order: the first one is innermost */
  int intl[MAX_IDX], nint = 0;
  for (int k = 0; k < s->rank[1]; k++) {
    int id = s->pos[1][k];
    if (occurs(s, 0, id) == 0) intl[nint++] = id;
  }
  for (int k = 0; k < nint; k++) digit[intl[k]] = 0;
  double sum = 0.0, comp = 0.0, abssum = 0.0;
  for (;;) {
    long long oa = 0, ob = 0;
    for (int id = 0; id < s->nidx; id++) {
      oa += digit[id] * s->stride[1][id];
      ob += digit[id] * s->stride[2][id];
    }
    double prod = load_elem(A, dtype, oa) * load_elem(B, dtype, ob);
    if (exact) {                          /* Neumaier */
      double t = sum + prod;
      if (fabs(sum) >= fabs(prod)) comp += (sum - t) + prod;
      else comp += (prod - t) + sum;
      sum = t;
    } else {
      sum = sum + prod;
    }
    abssum = abssum + fabs(prod);
    /* odometer over the internal indices */
    int k = 0;
    for (; k < nint; k++) {
      int id = intl[k];
      if (++digit[id] < s->ext[id]) break;
      digit[id] = 0;
    }
    if (k == nint) break;
  }
  if (exact) sum = sum + comp;
  double out = alpha * sum;
  double sc = fabs(alpha) * abssum;
  if (beta != 0.0) {
    double c = load_elem(Cin, dtype, x);
    out = out + beta * c;
    sc = sc + fabs(beta) * fabs(c);
  }
  *val = out;
  *scale = sc;
}

static int run(const char *expr, const char *extents, int dtype, const void *A, const void *B,
               const void *Cin, void *Cout, double *S, double alpha, double beta,
               const int64_t *idx, int64_t lo, int64_t n, int exact, int nthreads) {
  Spec s;
  int st = parse_all(&s, expr, extents);
  if (st) return st;
  if (dtype < 0 || dtype > 3) return E_UNSUP;
  if (!A || !B || !Cout || (beta != 0.0 && !Cin) || n < 0) return E_ARG;
  for (int64_t i = 0; i < n; i++) {
    long long x = idx ? idx[i] : lo + i;
    if (x < 0 || x >= s.numel[0]) return E_ARG;
  }
#ifdef _OPENMP
  int nt = nthreads > 0 ? nthreads : omp_get_max_threads();
#pragma omp parallel for schedule(dynamic, 64) num_threads(nt)
#endif
  for (int64_t i = 0; i < n; i++) {
    long long x = idx ? idx[i] : lo + i;
    double v, sc;
    one_element(&s, dtype, A, B, Cin, alpha, beta, x, exact, &v, &sc);
    store_elem(Cout, dtype, i, v);
    if (S) S[i] = sc;
  }
  (void)nthreads;
  return OK;
}

int tco_range(const char *expr, const char *extents, int dtype, const void *A, const void *B,
              const void *C_in, void *C_out, double *S_out, double alpha, double beta,
              int64_t lo, int64_t hi, int exact, int nthreads) {
  if (hi < lo) return E_ARG;
  return run(expr, extents, dtype, A, B, C_in, C_out, S_out, alpha, beta, NULL, lo, hi - lo,
             exact, nthreads);
}

int tco_sample(const char *expr, const char *extents, int dtype, const void *A, const void *B,
               const void *C_in, void *C_out, double *S_out, double alpha, double beta,
               const int64_t *idx, int64_t n, int exact, int nthreads) {
  if (!idx && n > 0) return E_ARG;
  return run(expr, extents, dtype, A, B, C_in, C_out, S_out, alpha, beta, idx, 0, n, exact,
             nthreads);
}
