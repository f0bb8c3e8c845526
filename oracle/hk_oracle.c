/*
 * HAUBERK CPU oracle — TEST INFRASTRUCTURE, NOT PART OF THE PRODUCT.
 *
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference legs may
 * load this library.  It shares no code, header, table or constant generator with the CUDA path
 * under paper_conf_ipps_yimpski11_b200/ (both are written independently from DESIGN.md §3,
 * which restates PAPER.md).  Plain, slow, single-threaded, obviously-correct C11:
 * compiled with -O2 -fno-fast-math -ffp-contract=off so every float operation is one IEEE-754
 * binary32 operation in the order written; fmaf() is the only fused operation and appears
 * exactly where DESIGN.md writes fmaf.
 *
 * Citations: "PAPER Lnnn" = /root/reference/PAPER.md line nnn (section in brackets);
 * "Rnn" = DESIGN.md reading nn (the paper's silent/ambiguous points).
 *
 * What is here, in the paper's order:
 *   - HAUBERK-NL: duplicate + compare + two-XOR checksum per virtual variable
 *     (PAPER L986-1042 [§V.A steps i-v]); kernel parameters XORed at entry/exit (L1045-1053);
 *     load duplication (L1199-1200).
 *   - HAUBERK-L: self-accumulator selection (L1221-1273 [§V.B step i]), accumulator and counter
 *     (L1275-1300 [steps ii-iii]), HauberkCheckRange / HauberkCheckEqual after the loop
 *     (L1302-1313, L1405-1429 [step iv]).
 *   - Value-range profiler with <= 3 correlation points (L1489-1508 [§V.B]), readings R8-R11.
 *   - Single-bit SWIFI at variable granularity (L2186-2272 [§VII]), readings R13-R18.
 *   - Outcome classes and coverage (L2370-2387 [§VIII]; L2480-2483), readings R1-R7.
 *   - The three benchmarks as plain definitions (double) and as the FP32 spec sequences of
 *     DESIGN.md §3.2-3.4 (CP: PAPER Fig. 9 L1242-1258 and the snippet at L1422-1429).
 *
 * Parity pins: see tests/test_oracle_*.py.  Functions without a pin say "parity unpinned".
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#define ORA_EXPORT __attribute__((visibility("default")))

/* ------------------------------------------------------------------------------------------ */
/* Shared enums (values fixed by DESIGN.md §3.1; the CUDA side declares its own copy)          */
/* ------------------------------------------------------------------------------------------ */
enum { B_CP = 0, B_MRIQ = 1, B_TPACF = 2 };
enum { C_MASKED = 0, C_DET_MASKED = 1, C_DETECTED = 2, C_UNDETECTED = 3, C_FAILURE = 4 };
enum { AL_DUP = 1, AL_CHK = 2, AL_RANGE = 4, AL_COUNT = 8 };
enum { FL_CRASH = 1, FL_HANG = 2 };
enum { F_NL = 1, F_L = 2, F_PROFILE = 4, F_FI = 8 };
enum { SC_NL = 0, SC_ITER = 1 }; /* NL @def: one instance per thread; else: golden-trip instances */

/* Canonical virtual base of every pointer parameter for the crash model (R16). */
static const uint64_t VBASE = 0x00007F0000000000ull;

typedef struct { int32_t n; float lo[3], hi[3]; int32_t t_exp10; } ora_rset;
typedef struct { int32_t n_det; float alpha; ora_rset det[8]; } ora_ranges;

typedef struct { const float* atoms; int32_t n_atoms; float z0, h; int32_t nx, ny, bx, by, unroll; } ora_cp_args;
typedef struct {
  const float *x, *y, *z; int32_t n_vox; int32_t n_k;
  const float *kx, *ky, *kz, *phi_r, *phi_i;
} ora_mriq_args;
typedef struct { const float* pts; const float* edges; int32_t n, n_rand, n_bins; } ora_tpacf_args;

/* hang = R17 watchdog factor T of this injection (0 = the paper's 10, L1997-2001). */
typedef struct { int32_t site; int32_t hang; int64_t thread, inst; uint64_t mask; } ora_fault;
typedef struct {
  uint32_t alarm, fail, domain, margin;
  uint32_t n_alarm_threads, first_thread; int32_t applied; float gap;
} ora_runinfo;
typedef struct {
  int64_t index; int32_t bench, site; int64_t thread, inst; uint64_t mask;
  int32_t cls; uint32_t alarm, fail, domain, margin; float worst; float gap; int32_t pad;
} ora_record;

/* ------------------------------------------------------------------------------------------ */
/* Bit helpers, wrapping int32 arithmetic (all i32 arithmetic is mod 2^32)     */
/* ------------------------------------------------------------------------------------------ */
static uint32_t fb(float f) { uint32_t u; memcpy(&u, &f, 4); return u; }
static float bf(uint32_t u) { float f; memcpy(&f, &u, 4); return f; }
static int32_t add32(int32_t a, int32_t b) { return (int32_t)((uint32_t)a + (uint32_t)b); }
static int32_t sub32(int32_t a, int32_t b) { return (int32_t)((uint32_t)a - (uint32_t)b); }
static int32_t mul32(int32_t a, int32_t b) { return (int32_t)((uint32_t)a * (uint32_t)b); }
static uint32_t lohi(uint64_t p) { return (uint32_t)p ^ (uint32_t)(p >> 32); }

/* R8: ordinal of a binary32 encoding; +0 and -0 both map to 0. */
ORA_EXPORT int64_t ora_ord(float x) {
  uint32_t b = fb(x);
  if (b & 0x80000000u) return -(int64_t)(b & 0x7fffffffu);
  return (int64_t)b;
}

/* ------------------------------------------------------------------------------------------ */
/* R15: stateless SplitMix64; output m of the stream seeded with `seed`.                       */
/* ------------------------------------------------------------------------------------------ */
ORA_EXPORT uint64_t ora_splitmix(uint64_t seed, uint64_t m) {
  uint64_t z = seed + (m + 1) * 0x9E3779B97F4A7C15ull;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}
ORA_EXPORT uint64_t ora_bounded(uint64_t r, uint64_t m) {
  return (uint64_t)(((unsigned __int128)r * (unsigned __int128)m) >> 64);
}

/* ------------------------------------------------------------------------------------------ */
/* Transcendentals (R20).  FAST = the value the GPU's MUFU approximates: correctly rounded      */
/* from double, with the MUFU special cases (.ftz input, 0 -> inf, <0 -> NaN, inf -> 0).        */
/* EXACT = a fixed FP32 op sequence reproduced bit-for-bit by both implementations.            */
/* ------------------------------------------------------------------------------------------ */
static int is_denorm(float x) { uint32_t b = fb(x) & 0x7fffffffu; return b != 0 && b < 0x00800000u; }

ORA_EXPORT float ora_rsqrt(float x, int32_t exact) {
  if (exact) {
    /* magic-constant seed + 3 Newton steps, R20 */
    float y = bf(0x5F375A86u - (fb(x) >> 1));
    float hx = 0.5f * x;
    for (int k = 0; k < 3; ++k) {
      float t = hx * y;
      t = fmaf(-t, y, 1.5f);
      y = y * t;
    }
    return y;
  }
  if (isnan(x)) return x;
  if (is_denorm(x)) x = signbit(x) ? -0.0f : 0.0f;
  if (x == 0.0f) return signbit(x) ? -INFINITY : INFINITY;
  if (x < 0.0f) return NAN;
  if (isinf(x)) return 0.0f;
  return (float)(1.0 / sqrt((double)x));
}

/* EXACT sin/cos: Taylor polynomials in a^2, coefficients (float)(+-1/n!) (R20). */
static float sin_coef(int k) { double f = 1.0; for (int i = 2; i <= 2 * k + 1; ++i) f *= i; return (float)((k & 1) ? -1.0 / f : 1.0 / f); }
static float cos_coef(int k) { double f = 1.0; for (int i = 2; i <= 2 * k; ++i) f *= i; return (float)((k & 1) ? -1.0 / f : 1.0 / f); }

ORA_EXPORT float ora_cos(float a, int32_t exact) {
  if (exact) {
    float s2 = a * a;
    float q = cos_coef(10);
    for (int k = 9; k >= 0; --k) q = fmaf(q, s2, cos_coef(k));
    return q;
  }
  if (is_denorm(a)) a = 0.0f;
  if (!isfinite(a)) return NAN;
  return (float)cos((double)a);
}
ORA_EXPORT float ora_sin(float a, int32_t exact) {
  if (exact) {
    float s2 = a * a;
    float p = sin_coef(9);
    for (int k = 8; k >= 0; --k) p = fmaf(p, s2, sin_coef(k));
    return a * p;
  }
  if (is_denorm(a)) a = signbit(a) ? -0.0f : 0.0f;
  if (!isfinite(a)) return NAN;
  return (float)sin((double)a);
}

/* ------------------------------------------------------------------------------------------ */
/* Fault context: one flip of one site at one dynamic instance of one thread (R13).            */
/* ------------------------------------------------------------------------------------------ */
typedef struct {
  int active;      /* this thread is the injection target */
  int site;
  int64_t inst;
  uint64_t mask;
  int applied;
  int32_t hang;    /* R17 watchdog factor T ("T (i.e., 10) times") */
} fctx;

/* R17: a loop about to start iteration `it` >= T * max(golden trips, 1) is FAILURE(hang).  The
 * limit comes from the fault-free trip count known to the harness (not from corruptible state). */
static int64_t hang_limit(const fctx* F, int64_t golden) {
  const int64_t T = (F && F->hang > 0) ? F->hang : 10;
  return T * (golden > 1 ? golden : 1);
}

static int hit(fctx* F, int site, int64_t inst) {
  if (F && F->active && F->site == site && F->inst == inst) { F->applied = 1; return 1; }
  return 0;
}
static int32_t fi32(fctx* F, int site, int64_t inst, int32_t v) { return hit(F, site, inst) ? (int32_t)((uint32_t)v ^ (uint32_t)F->mask) : v; }
static float ff32(fctx* F, int site, int64_t inst, float v) { return hit(F, site, inst) ? bf(fb(v) ^ (uint32_t)F->mask) : v; }
static uint64_t fp64(fctx* F, int site, int64_t inst, uint64_t v) { return hit(F, site, inst) ? v ^ F->mask : v; }

/* R16 crash model: element access through a (possibly flipped) pointer parameter.
 * Returns 1 and the element index if in bounds, 0 on a modelled crash. */
static int access_ok(uint64_t ptr, int32_t idx, int64_t esz, int64_t n, int64_t* e) {
  int64_t delta = (int64_t)(ptr - VBASE);
  if (delta % esz != 0) return 0;
  int64_t ei = (int64_t)idx + delta / esz;
  if (ei < 0 || ei >= n) return 0;
  *e = ei;
  return 1;
}

/* R10/R11: alpha-widened range check; NaN is out of range. */
static float lo_alpha(float lo, float a) { return lo > 0.0f ? lo / a : lo * a; }
static float hi_alpha(float hi, float a) { return hi > 0.0f ? hi * a : hi / a; }
static uint32_t ord_dist(float a, float b) {
  int64_t d = ora_ord(a) - ora_ord(b);
  if (d < 0) d = -d;
  return d > 0x7fffffff ? 0x7fffffffu : (uint32_t)d;
}
/* Returns 1 if in range.  Updates *margin with the min ordinal distance to any bound and *gap with
 * the min absolute distance |v - bound| (the two measures of the R22(a) guard band). */
static int in_range(const ora_ranges* R, int d, float v, uint32_t* margin, float* gap) {
  const ora_rset* s = &R->det[d];
  int in = 0;
  for (int r = 0; r < s->n; ++r) {
    float lo = lo_alpha(s->lo[r], R->alpha), hi = hi_alpha(s->hi[r], R->alpha);
    if (lo <= v && v <= hi) in = 1;
    if (!isnan(v)) {
      uint32_t a = ord_dist(v, lo), b = ord_dist(v, hi);
      if (a < *margin) *margin = a;
      if (b < *margin) *margin = b;
      float ga = fabsf(v - lo), gb = fabsf(v - hi);
      if (ga < *gap) *gap = ga;
      if (gb < *gap) *gap = gb;
    }
  }
  return in;
}

typedef struct {
  uint32_t alarm, fail, domain, margin; float gap;
  int nw; int32_t wbuf[16]; int64_t widx[16]; float wval[16];
} tout;

static void tout_init(tout* o) { memset(o, 0, sizeof(*o)); o->margin = 0xffffffffu; o->gap = INFINITY; }

/* ------------------------------------------------------------------------------------------ */
/* CP (K1).  DESIGN.md §3.2; PAPER Fig. 9, loop-detector code L1422-1429.           */
/* Site catalogue (U = unroll):                                                                */
/*   0 xindex 1 yindex 2 outaddr 3 coorx 4 coory 5 gu                  (NL @def)               */
/*   6 outaddr 7 coorx 8 coory 9 gu                                     (NL @live)             */
/*   10 numatoms 11 h 12 grid* 13 atoms*                                (param @live; * = 64b) */
/*   14 atomid 15 ax 16 ay 17 az 18 aw 19 dy 20 dyz2 21 dx0             (loop @def)            */
/*   22..20+U dx_j (j=1..U-1); then r2_j (U), s_j (U), E_j (U, @acc), it (@acc)               */
/* ------------------------------------------------------------------------------------------ */
static int cp_nsites(int U) { return 22 + 4 * U; }
/* Detector d's self-accumulator (A6 repeated Maxvar times, L1259-1273; pinned by ora_a6_select on
 * the CP loop graph): E_{U-1} first (largest backward dependency: it chains every dx_j), then the
 * remaining E_j tie at {r2_j, s_j} and go in program order E_0, E_1, ... (R12). */
static int cp_sel(int U, int d) { return d == 0 ? U - 1 : d - 1; }

static void cp_thread(const ora_cp_args* P, const float* A4, int64_t t, int flags, int exact,
                      const ora_ranges* R, int ndet, fctx* F, tout* o, float* samples, int64_t nthr) {
  const int U = P->unroll, BX = P->bx, BY = P->by;
  const int nbx = P->nx / (BX * U);
  const int64_t per_blk = (int64_t)BX * BY;
  const int64_t blk = t / per_blk;
  const int tx = (int)((t % per_blk) % BX), ty = (int)((t % per_blk) / BX);
  const int bxi = (int)(blk % nbx), byi = (int)(blk / nbx);
  const int NL = flags & F_NL, L = flags & F_L, FI = flags & F_FI;
  const int S_DX = 22, S_R2 = 22 + (U - 1), S_S = S_R2 + U, S_E = S_S + U, S_IT = S_E + U;

  uint32_t chk = 0;
  int32_t numatoms = P->n_atoms;
  float h = P->h;
  uint64_t pgrid = VBASE, patoms = VBASE;
  if (NL) { chk ^= (uint32_t)numatoms; chk ^= fb(h); chk ^= lohi(pgrid); chk ^= lohi(patoms); }

  /* Non-loop virtual variables: def, [flip], (i) chk ^= v, (ii) duplicate, (iii) compare. */
  int32_t xindex = add32(mul32(bxi, BX * U), tx);
  xindex = fi32(F, 0, 0, xindex);
  if (NL) { chk ^= (uint32_t)xindex; if (add32(mul32(bxi, BX * U), tx) != xindex) o->alarm |= AL_DUP; }
  int32_t yindex = add32(mul32(byi, BY), ty);
  yindex = fi32(F, 1, 0, yindex);
  if (NL) { chk ^= (uint32_t)yindex; if (add32(mul32(byi, BY), ty) != yindex) o->alarm |= AL_DUP; }
  const int32_t nx = nbx * BX * U;
  int32_t outaddr = add32(mul32(nx, yindex), xindex);
  outaddr = fi32(F, 2, 0, outaddr);
  if (NL) { chk ^= (uint32_t)outaddr; if (add32(mul32(nx, yindex), xindex) != outaddr) o->alarm |= AL_DUP; }
  float coorx = h * (float)xindex;
  coorx = ff32(F, 3, 0, coorx);
  if (NL) { chk ^= fb(coorx); if (fb(h * (float)xindex) != fb(coorx)) o->alarm |= AL_DUP; }
  float coory = h * (float)yindex;
  coory = ff32(F, 4, 0, coory);
  if (NL) { chk ^= fb(coory); if (fb(h * (float)yindex) != fb(coory)) o->alarm |= AL_DUP; }
  float gu = h * (float)BX;
  gu = ff32(F, 5, 0, gu);
  if (NL) { chk ^= fb(gu); if (fb(h * (float)BX) != fb(gu)) o->alarm |= AL_DUP; }
  /* (iv) xindex, yindex: last use was above (not used in the loop). */
  if (NL) { chk ^= (uint32_t)xindex; chk ^= (uint32_t)yindex; }

  /* Loop (self-accumulators E_j need no accumulator; counter `it`). */
  float E[8] = {0};
  int32_t it = 0;
  const int64_t limit = hang_limit(F, P->n_atoms);
  int32_t atomid = 0;
  for (int64_t i = 0;; ++i) {
    atomid = fi32(F, 14, i, atomid);
    outaddr = fi32(F, 6, i, outaddr);
    coorx = ff32(F, 7, i, coorx);
    coory = ff32(F, 8, i, coory);
    gu = ff32(F, 9, i, gu);
    numatoms = fi32(F, 10, i, numatoms);
    h = ff32(F, 11, i, h);
    pgrid = fp64(F, 12, i, pgrid);
    patoms = fp64(F, 13, i, patoms);
    if (!(atomid < numatoms)) break;
    if (FI && i >= limit) { o->fail |= FL_HANG; return; }
    int64_t e;
    if (FI) { if (!access_ok(patoms, atomid, 16, P->n_atoms, &e)) { o->fail |= FL_CRASH; return; } }
    else e = atomid;
    float ax = ff32(F, 15, i, A4[4 * e + 0]);
    float ay = ff32(F, 16, i, A4[4 * e + 1]);
    float az = ff32(F, 17, i, A4[4 * e + 2]);
    float aw = ff32(F, 18, i, A4[4 * e + 3]);
    float dy = ff32(F, 19, i, coory - ay);
    float dyz2 = ff32(F, 20, i, fmaf(dy, dy, az));
    float dx[8];
    dx[0] = ff32(F, 21, i, coorx - ax);
    for (int j = 1; j < U; ++j) dx[j] = ff32(F, S_DX + j - 1, i, dx[j - 1] + gu);
    for (int j = 0; j < U; ++j) {
      float r2 = ff32(F, S_R2 + j, i, fmaf(dx[j], dx[j], dyz2));
      float s = ff32(F, S_S + j, i, ora_rsqrt(r2, exact));
      E[j] = ff32(F, S_E + j, i, fmaf(aw, s, E[j]));
    }
    it = fi32(F, S_IT, i, add32(it, 1));
    atomid = add32(atomid, 1);
  }
  /* HauberkCheckEqual(it, numatoms), HauberkCheckRange(E_sel / it) */
  if (L && it != numatoms) o->alarm |= AL_COUNT;
  if ((L || (flags & F_PROFILE)) && it != 0) {
    for (int d = 0; d < ndet; ++d) {
      float v = E[cp_sel(U, d)] / (float)it;
      if (flags & F_PROFILE) samples[(int64_t)d * nthr + t] = v;
      if (L && R->det[d].n > 0 && !in_range(R, d, v, &o->margin, &o->gap)) o->alarm |= AL_RANGE;
    }
  }
  if (NL) { chk ^= fb(coorx); chk ^= fb(coory); chk ^= fb(gu); }
  for (int j = 0; j < U; ++j) {
    int32_t idx = add32(outaddr, j * BX);
    int64_t e;
    if (FI) { if (!access_ok(pgrid, idx, 4, (int64_t)P->nx * P->ny, &e)) { o->fail |= FL_CRASH; return; } }
    else e = idx;
    o->wbuf[o->nw] = 0; o->widx[o->nw] = e; o->wval[o->nw] = E[j]; o->nw++;
  }
  if (NL) {
    chk ^= (uint32_t)outaddr;
    chk ^= (uint32_t)numatoms; chk ^= fb(h); chk ^= lohi(pgrid); chk ^= lohi(patoms);
    if (chk != 0) o->alarm |= AL_CHK;
  }
}

/* Uninstrumented pre-pass (row a1): (x, y, z, q) -> (x, y, dz^2, q), dz = z - z0. */
static float* cp_prepass(const ora_cp_args* P) {
  float* A4 = (float*)malloc(sizeof(float) * 4 * (size_t)(P->n_atoms > 0 ? P->n_atoms : 1));
  for (int a = 0; a < P->n_atoms; ++a) {
    float dz = P->atoms[4 * a + 2] - P->z0;
    A4[4 * a + 0] = P->atoms[4 * a + 0];
    A4[4 * a + 1] = P->atoms[4 * a + 1];
    A4[4 * a + 2] = dz * dz;
    A4[4 * a + 3] = P->atoms[4 * a + 3];
  }
  return A4;
}

static int64_t cp_threads(const ora_cp_args* P) { return (int64_t)(P->nx / P->unroll) * P->ny; }

static int cp_valid(const ora_cp_args* P) {
  if (P->unroll < 1 || P->unroll > 8 || P->bx < 1 || P->by < 1) return 0;
  if (P->nx % (P->bx * P->unroll) != 0 || P->ny % P->by != 0 || P->n_atoms < 0) return 0;
  return 1;
}

/* ------------------------------------------------------------------------------------------ */
/* MRI-Q (K2).  DESIGN.md §3.3.  PhiMag: pm = fmaf(im, im, re*re); Q loop per voxel.            */
/* Q-kernel site catalogue:                                                                    */
/*   0 xIndex 1 sX 2 sY 3 sZ (NL @def) 4 xIndex 5 sX 6 sY 7 sZ (NL @live)                      */
/*   8 numK 9 kv* 10 qr* 11 qi* 12 x* 13 y* 14 z* (param @live)                                */
/*   15 k 16 kx 17 ky 18 kz 19 pm 20 t1 21 t2 22 t 23 r 24 c 25 s 26 Qr 27 Qi 28 it (loop)     */
/* ------------------------------------------------------------------------------------------ */
#define MRIQ_NSITES 36
#define MRIQ_PHIMAG_SITE0 29 /* 29 kidx 30 re 31 im 32 pm 33 kx 34 ky 35 kz: PhiMag NL @def (replica only) */
static const float TWO_PI_F = 6.28318548202514648f; /* binary32 nearest 2*pi (0x40C90FDB) */
static const float RINT_MAGIC = 12582912.0f;        /* 1.5 * 2^23 */

/* PhiMag abstract thread k (non-loop code: HAUBERK-NL on every virtual variable, loads included,
 * A1-A3).  kv is written additively into a zeroed buffer (R18).  Sites 29-35. */
static void phimag_thread(const ora_mriq_args* P, int64_t k, int flags, fctx* F, tout* o, float* kv) {
  const int NL = flags & F_NL, FI = flags & F_FI;
  uint32_t chk = 0;
  const int64_t nk = P->n_k;
  int64_t e;
  int32_t kidx = fi32(F, 29, 0, (int32_t)k);
  if (NL) { chk ^= (uint32_t)kidx; if ((int32_t)k != kidx) o->alarm |= AL_DUP; }
#define PHLOAD(var, arr, site)                                                       \
  if (FI && !access_ok(VBASE, kidx, 4, nk, &e)) { o->fail |= FL_CRASH; return; }      \
  else if (!FI) e = kidx;                                                           \
  float var = ff32(F, site, 0, (arr)[e]);                                           \
  if (NL) { chk ^= fb(var); if (fb((arr)[e]) != fb(var)) o->alarm |= AL_DUP; }
  PHLOAD(re, P->phi_r, 30)
  PHLOAD(im, P->phi_i, 31)
  float pm = ff32(F, 32, 0, fmaf(im, im, re * re));
  if (NL) { chk ^= fb(pm); if (fb(fmaf(im, im, re * re)) != fb(pm)) o->alarm |= AL_DUP; }
  PHLOAD(kx, P->kx, 33)
  PHLOAD(ky, P->ky, 34)
  PHLOAD(kz, P->kz, 35)
#undef PHLOAD
  if (FI && !access_ok(VBASE, kidx, 16, nk, &e)) { o->fail |= FL_CRASH; return; }
  else if (!FI) e = kidx;
  kv[4 * e + 0] = kv[4 * e + 0] + kx;
  kv[4 * e + 1] = kv[4 * e + 1] + ky;
  kv[4 * e + 2] = kv[4 * e + 2] + kz;
  kv[4 * e + 3] = kv[4 * e + 3] + pm;
  if (NL) {
    chk ^= fb(re); chk ^= fb(im); chk ^= fb(pm); chk ^= fb(kx); chk ^= fb(ky); chk ^= fb(kz); chk ^= (uint32_t)kidx;
    if (chk != 0) o->alarm |= AL_CHK;
  }
}

static float* mriq_phimag(const ora_mriq_args* P) {
  float* kv = (float*)malloc(sizeof(float) * 4 * (size_t)(P->n_k > 0 ? P->n_k : 1));
  for (int k = 0; k < P->n_k; ++k) {
    float re = P->phi_r[k], im = P->phi_i[k];
    kv[4 * k + 0] = P->kx[k];
    kv[4 * k + 1] = P->ky[k];
    kv[4 * k + 2] = P->kz[k];
    kv[4 * k + 3] = fmaf(im, im, re * re);
  }
  return kv;
}

static void mriq_thread(const ora_mriq_args* P, const float* KV, int64_t t, int flags, int exact,
                        const ora_ranges* R, int ndet, fctx* F, tout* o, float* samples, int64_t nthr) {
  const int NL = flags & F_NL, L = flags & F_L, FI = flags & F_FI;
  uint32_t chk = 0;
  int32_t numK = P->n_k;
  uint64_t pkv = VBASE, pqr = VBASE, pqi = VBASE, px = VBASE, py = VBASE, pz = VBASE;
  if (NL) { chk ^= (uint32_t)numK; chk ^= lohi(pkv) ^ lohi(pqr) ^ lohi(pqi) ^ lohi(px) ^ lohi(py) ^ lohi(pz); }

  int32_t xIndex = (int32_t)t;
  xIndex = fi32(F, 0, 0, xIndex);
  if (NL) { chk ^= (uint32_t)xIndex; if ((int32_t)t != xIndex) o->alarm |= AL_DUP; }
  int64_t e;
  const int64_t nv = P->n_vox;
  float sX, sY, sZ;
  if (FI && !access_ok(px, xIndex, 4, nv, &e)) { o->fail |= FL_CRASH; return; } else e = (FI ? e : xIndex);
  sX = ff32(F, 1, 0, P->x[e]);
  if (NL) { chk ^= fb(sX); if (fb(P->x[e]) != fb(sX)) o->alarm |= AL_DUP; }
  if (FI && !access_ok(py, xIndex, 4, nv, &e)) { o->fail |= FL_CRASH; return; } else e = (FI ? e : xIndex);
  sY = ff32(F, 2, 0, P->y[e]);
  if (NL) { chk ^= fb(sY); if (fb(P->y[e]) != fb(sY)) o->alarm |= AL_DUP; }
  if (FI && !access_ok(pz, xIndex, 4, nv, &e)) { o->fail |= FL_CRASH; return; } else e = (FI ? e : xIndex);
  sZ = ff32(F, 3, 0, P->z[e]);
  if (NL) { chk ^= fb(sZ); if (fb(P->z[e]) != fb(sZ)) o->alarm |= AL_DUP; }

  float Qr = 0.0f, Qi = 0.0f;
  int32_t it = 0, k = 0;
  const int64_t limit = hang_limit(F, P->n_k);
  for (int64_t i = 0;; ++i) {
    k = fi32(F, 15, i, k);
    xIndex = fi32(F, 4, i, xIndex);
    sX = ff32(F, 5, i, sX); sY = ff32(F, 6, i, sY); sZ = ff32(F, 7, i, sZ);
    numK = fi32(F, 8, i, numK);
    pkv = fp64(F, 9, i, pkv); pqr = fp64(F, 10, i, pqr); pqi = fp64(F, 11, i, pqi);
    px = fp64(F, 12, i, px); py = fp64(F, 13, i, py); pz = fp64(F, 14, i, pz);
    if (!(k < numK)) break;
    if (FI && i >= limit) { o->fail |= FL_HANG; return; }
    if (FI) { if (!access_ok(pkv, k, 16, P->n_k, &e)) { o->fail |= FL_CRASH; return; } }
    else e = k;
    float kx = ff32(F, 16, i, KV[4 * e + 0]);
    float ky = ff32(F, 17, i, KV[4 * e + 1]);
    float kz = ff32(F, 18, i, KV[4 * e + 2]);
    float pm = ff32(F, 19, i, KV[4 * e + 3]);
    float t1 = ff32(F, 20, i, kx * sX);
    float t2 = ff32(F, 21, i, fmaf(ky, sY, t1));
    float tt = ff32(F, 22, i, fmaf(kz, sZ, t2));
    float m = (tt + RINT_MAGIC) - RINT_MAGIC; /* rint(tt) for |tt| < 2^22 */
    float r = ff32(F, 23, i, tt - m);
    if (!exact && isfinite(r) && fabsf(r) > 0.5f) o->domain = 1;
    float ang = r * TWO_PI_F;
    float c = ff32(F, 24, i, ora_cos(ang, exact));
    float s = ff32(F, 25, i, ora_sin(ang, exact));
    Qr = ff32(F, 26, i, fmaf(pm, c, Qr));
    Qi = ff32(F, 27, i, fmaf(pm, s, Qi));
    it = fi32(F, 28, i, add32(it, 1));
    k = add32(k, 1);
  }
  if (L && it != numK) o->alarm |= AL_COUNT;
  if ((L || (flags & F_PROFILE)) && it != 0) {
    for (int d = 0; d < ndet; ++d) {
      float v = (d == 0 ? Qr : Qi) / (float)it;
      if (flags & F_PROFILE) samples[(int64_t)d * nthr + t] = v;
      if (L && R->det[d].n > 0 && !in_range(R, d, v, &o->margin, &o->gap)) o->alarm |= AL_RANGE;
    }
  }
  if (NL) { chk ^= fb(sX); chk ^= fb(sY); chk ^= fb(sZ); }
  if (FI) { if (!access_ok(pqr, xIndex, 4, nv, &e)) { o->fail |= FL_CRASH; return; } } else e = xIndex;
  o->wbuf[o->nw] = 0; o->widx[o->nw] = e; o->wval[o->nw] = Qr; o->nw++;
  if (FI) { if (!access_ok(pqi, xIndex, 4, nv, &e)) { o->fail |= FL_CRASH; return; } } else e = xIndex;
  o->wbuf[o->nw] = 1; o->widx[o->nw] = e; o->wval[o->nw] = Qi; o->nw++;
  if (NL) {
    chk ^= (uint32_t)xIndex;
    chk ^= (uint32_t)numK; chk ^= lohi(pkv) ^ lohi(pqr) ^ lohi(pqi) ^ lohi(px) ^ lohi(py) ^ lohi(pz);
    if (chk != 0) o->alarm |= AL_CHK;
  }
}

static int mriq_valid(const ora_mriq_args* P) { return P->n_vox >= 0 && P->n_k >= 0; }

/* ------------------------------------------------------------------------------------------ */
/* TPACF (K3).  DESIGN.md §3.4: one abstract thread g = h*N + i per (histogram */
/* h, point i), looping over every partner j in [jb, N) in ascending order.  There is no chunk  */
/* here: how a kernel tiles the partner loop is not part of the program.                       */
/* Site catalogue:                                                                             */
/*   0 i 1 h 2 aoff 3 boff 4 jb 5 je 6 expect 7 base 8 x1 9 y1 10 z1          (NL @def)        */
/*   11 boff 12 je 13 expect 14 base 15 x1 16 y1 17 z1                        (NL @live)       */
/*   18 n 19 pts* 20 hist*                                                   (param @live)    */
/*   21 j 22 x2 23 y2 24 z2 25 dot 26 bin 27 hidx 28 acc 29 cnt               (loop)           */
/* ------------------------------------------------------------------------------------------ */
#define TPACF_NSITES 30
static int tp_nh(const ora_tpacf_args* P) { return 1 + 2 * P->n_rand; }
static int64_t tp_threads(const ora_tpacf_args* P) { return (int64_t)tp_nh(P) * P->n; }
static int tp_valid(const ora_tpacf_args* P) {
  if (P->n < 0 || P->n_rand < 1 || P->n_bins < 1 || P->n_bins > 30) return 0;
  for (int e = 0; e < P->n_bins; ++e) if (!(P->edges[e] > P->edges[e + 1])) return 0;
  return 1;
}
/* Golden trip count of thread g (computed from uncorrupted indices; R17 watchdog, decode):
 * N - (i + 1) for the self-correlation rows h <= n_rand (DD, RR_s), N for the DR rows. */
static int64_t tp_trips(const ora_tpacf_args* P, int64_t g) {
  int64_t h = g / P->n, i = g % P->n;
  return h <= P->n_rand ? (int64_t)P->n - (i + 1) : (int64_t)P->n;
}
/* bin = #{e in [0, n_bins] : dot < edge[e]}  (the definition) */
static int32_t tp_bin(const ora_tpacf_args* P, float dot) {
  int32_t b = 0;
  for (int e = 0; e <= P->n_bins; ++e) if (dot < P->edges[e]) b++;
  return b;
}

static void tpacf_thread(const ora_tpacf_args* P, int64_t g, int flags, const ora_ranges* R, int ndet,
                         fctx* F, tout* o, int64_t* hist, float* samples, int64_t nthr) {
  const int NL = flags & F_NL, L = flags & F_L, FI = flags & F_FI;
  const int nr = P->n_rand, nb2 = P->n_bins + 2;
  const int64_t npts = 3LL * (1 + nr) * P->n, nhist = (int64_t)tp_nh(P) * nb2;
  const int32_t hh = (int32_t)(g / P->n), ii = (int32_t)(g % P->n);
  uint32_t chk = 0;
  int32_t n = P->n;
  uint64_t ppts = VBASE, phist = VBASE;
  if (NL) { chk ^= (uint32_t)n; chk ^= lohi(ppts); chk ^= lohi(phist); }

#define NLDEF(var, site, expr)                                              \
  var = fi32(F, site, 0, (expr));                                           \
  if (NL) { chk ^= (uint32_t)var; if ((expr) != var) o->alarm |= AL_DUP; }
  int32_t i, h, aoff, boff, jb, je, expect, base;
  NLDEF(i, 0, ii);
  NLDEF(h, 1, hh);
  NLDEF(aoff, 2, add32(mul32(h <= nr ? h : 0, n), i));
  NLDEF(boff, 3, mul32(h == 0 ? 0 : (h <= nr ? h : sub32(h, nr)), n));
  NLDEF(jb, 4, (h <= nr ? add32(i, 1) : 0));
  NLDEF(je, 5, n);
  NLDEF(expect, 6, (sub32(je, jb) > 0 ? sub32(je, jb) : 0));
  NLDEF(base, 7, mul32(h, nb2));
#undef NLDEF
  int64_t e;
  float x1, y1, z1;
  if (FI && !access_ok(ppts, add32(mul32(3, aoff), 0), 4, npts, &e)) { o->fail |= FL_CRASH; return; } else if (!FI) e = 3LL * aoff + 0;
  x1 = ff32(F, 8, 0, P->pts[e]);
  if (NL) { chk ^= fb(x1); if (fb(P->pts[e]) != fb(x1)) o->alarm |= AL_DUP; }
  if (FI && !access_ok(ppts, add32(mul32(3, aoff), 1), 4, npts, &e)) { o->fail |= FL_CRASH; return; } else if (!FI) e = 3LL * aoff + 1;
  y1 = ff32(F, 9, 0, P->pts[e]);
  if (NL) { chk ^= fb(y1); if (fb(P->pts[e]) != fb(y1)) o->alarm |= AL_DUP; }
  if (FI && !access_ok(ppts, add32(mul32(3, aoff), 2), 4, npts, &e)) { o->fail |= FL_CRASH; return; } else if (!FI) e = 3LL * aoff + 2;
  z1 = ff32(F, 10, 0, P->pts[e]);
  if (NL) { chk ^= fb(z1); if (fb(P->pts[e]) != fb(z1)) o->alarm |= AL_DUP; }
  /* (iv) for variables whose last use precedes the loop */
  if (NL) { chk ^= (uint32_t)i; chk ^= (uint32_t)h; chk ^= (uint32_t)aoff; chk ^= (uint32_t)jb; }

  int32_t acc = 0, cnt = 0, j = jb;
  const int64_t limit = hang_limit(F, tp_trips(P, g));
  for (int64_t it = 0;; ++it) {
    j = fi32(F, 21, it, j);
    boff = fi32(F, 11, it, boff); je = fi32(F, 12, it, je); expect = fi32(F, 13, it, expect);
    base = fi32(F, 14, it, base);
    x1 = ff32(F, 15, it, x1); y1 = ff32(F, 16, it, y1); z1 = ff32(F, 17, it, z1);
    n = fi32(F, 18, it, n); ppts = fp64(F, 19, it, ppts); phist = fp64(F, 20, it, phist);
    if (!(j < je)) break;
    if (FI && it >= limit) { o->fail |= FL_HANG; return; }
    int32_t pb = mul32(3, add32(boff, j));
    float q[3];
    for (int a = 0; a < 3; ++a) {
      if (FI) { if (!access_ok(ppts, add32(pb, a), 4, npts, &e)) { o->fail |= FL_CRASH; return; } }
      else e = (int64_t)pb + a;
      q[a] = ff32(F, 22 + a, it, P->pts[e]);
    }
    float dot = ff32(F, 25, it, fmaf(z1, q[2], fmaf(y1, q[1], x1 * q[0])));
    int32_t bin = fi32(F, 26, it, tp_bin(P, dot));
    int32_t hidx = fi32(F, 27, it, add32(base, bin));
    if (FI) { if (!access_ok(phist, hidx, 8, nhist, &e)) { o->fail |= FL_CRASH; return; } }
    else e = hidx;
    hist[e] += 1;
    acc = fi32(F, 28, it, add32(acc, bin));
    cnt = fi32(F, 29, it, add32(cnt, 1));
    j = add32(j, 1);
  }
  if (L && cnt != expect) o->alarm |= AL_COUNT;
  if ((L || (flags & F_PROFILE)) && cnt != 0 && ndet > 0) {
    float v = (float)acc / (float)cnt;
    if (flags & F_PROFILE) samples[g] = v;
    if (L && R->det[0].n > 0 && !in_range(R, 0, v, &o->margin, &o->gap)) o->alarm |= AL_RANGE;
  }
  if (NL) {
    chk ^= (uint32_t)boff; chk ^= (uint32_t)je; chk ^= (uint32_t)base;
    chk ^= fb(x1); chk ^= fb(y1); chk ^= fb(z1); chk ^= (uint32_t)expect;
    chk ^= (uint32_t)n; chk ^= lohi(ppts); chk ^= lohi(phist);
    if (chk != 0) o->alarm |= AL_CHK;
  }
}

/* ------------------------------------------------------------------------------------------ */
/* Full-program runs (replica mode): every abstract thread, at most one with a fault.          */
/* ------------------------------------------------------------------------------------------ */
static void info_fold(ora_runinfo* I, const tout* o, int64_t t, int target) {
  if (o->alarm) {
    I->alarm |= o->alarm;
    I->n_alarm_threads++;
    if ((uint32_t)t < I->first_thread) I->first_thread = (uint32_t)t;
  }
  I->fail |= o->fail;
  if (target) { I->domain |= o->domain; I->margin = o->margin; I->gap = o->gap; }
}
static void info_init(ora_runinfo* I) {
  memset(I, 0, sizeof(*I)); I->first_thread = 0xffffffffu; I->margin = 0xffffffffu; I->gap = INFINITY;
}

static fctx mkfctx(const ora_fault* f, int64_t t) {
  fctx F = {0, -1, 0, 0, 0, 10};
  if (f && f->site >= 0 && f->thread == t) { F.active = 1; F.site = f->site; F.inst = f->inst; F.mask = f->mask; }
  if (f && f->hang > 0) F.hang = f->hang;
  return F;
}

ORA_EXPORT int ora_cp_run(const ora_cp_args* P, int32_t flags, int32_t exact, const ora_ranges* R, int32_t ndet,
                          const ora_fault* f, float* grid, float* samples, ora_runinfo* I) {
  if (!cp_valid(P) || ndet < 0 || ndet > P->unroll) return 1;
  if (f && f->site >= 0) flags |= F_FI;
  float* A4 = cp_prepass(P);
  const int64_t nthr = cp_threads(P);
  memset(grid, 0, sizeof(float) * (size_t)P->nx * P->ny);
  info_init(I);
  for (int64_t t = 0; t < nthr; ++t) {
    fctx F = mkfctx(f, t);
    tout o; tout_init(&o);
    cp_thread(P, A4, t, flags, exact, R, ndet, &F, &o, samples, nthr);
    for (int w = 0; w < o.nw; ++w) grid[o.widx[w]] = grid[o.widx[w]] + o.wval[w]; /* R18 additive */
    info_fold(I, &o, t, F.active);
    if (F.active) I->applied = F.applied;
  }
  free(A4);
  return 0;
}

ORA_EXPORT int ora_mriq_run(const ora_mriq_args* P, int32_t flags, int32_t exact, const ora_ranges* R, int32_t ndet,
                            const ora_fault* f, float* qr, float* qi, float* samples, ora_runinfo* I) {
  if (!mriq_valid(P) || ndet < 0 || ndet > 2) return 1;
  if (f && f->site >= 0) flags |= F_FI;
  const int phimag_fault = f && f->site >= MRIQ_PHIMAG_SITE0;
  memset(qr, 0, sizeof(float) * (size_t)P->n_vox);
  memset(qi, 0, sizeof(float) * (size_t)P->n_vox);
  info_init(I);
  /* PhiMag (its detectors fold into the same control block as the Q kernel's) */
  float* KV = (float*)calloc(4 * (size_t)(P->n_k > 0 ? P->n_k : 1), sizeof(float));
  for (int64_t k = 0; k < P->n_k; ++k) {
    fctx F = phimag_fault ? mkfctx(f, k) : mkfctx(NULL, k);
    tout o; tout_init(&o);
    phimag_thread(P, k, flags & (F_NL | F_FI), &F, &o, KV);
    if (o.alarm || o.fail) { I->alarm |= o.alarm; I->fail |= o.fail; if (o.alarm) I->n_alarm_threads++; }
    if (F.active) I->applied = F.applied;
  }
  for (int64_t t = 0; t < P->n_vox; ++t) {
    fctx F = phimag_fault ? mkfctx(NULL, t) : mkfctx(f, t);
    tout o; tout_init(&o);
    mriq_thread(P, KV, t, flags, exact, R, ndet, &F, &o, samples, P->n_vox);
    for (int w = 0; w < o.nw; ++w) {
      float* buf = o.wbuf[w] ? qi : qr;
      buf[o.widx[w]] = buf[o.widx[w]] + o.wval[w];
    }
    info_fold(I, &o, t, F.active);
    if (F.active) I->applied = F.applied;
  }
  free(KV);
  return 0;
}

ORA_EXPORT int ora_tpacf_run(const ora_tpacf_args* P, int32_t flags, const ora_ranges* R, int32_t ndet,
                             const ora_fault* f, int64_t* hist, float* samples, ora_runinfo* I) {
  if (!tp_valid(P) || ndet < 0 || ndet > 1) return 1;
  if (f && f->site >= 0) flags |= F_FI;
  const int64_t nthr = tp_threads(P);
  memset(hist, 0, sizeof(int64_t) * (size_t)tp_nh(P) * (P->n_bins + 2));
  info_init(I);
  for (int64_t g = 0; g < nthr; ++g) {
    fctx F = mkfctx(f, g);
    tout o; tout_init(&o);
    tpacf_thread(P, g, flags, R, ndet, &F, &o, hist, samples, nthr);
    info_fold(I, &o, g, F.active);
    if (F.active) I->applied = F.applied;
  }
  return 0;
}

/* Outputs of single abstract threads (for sampled parity at full sizes): CP writes U values per
 * thread (grid index, value); MRI-Q writes (Qr, Qi) of each voxel. */
ORA_EXPORT int ora_cp_threads_out(const ora_cp_args* P, int32_t exact, const int64_t* tids, int64_t n, int64_t* idx, float* val) {
  if (!cp_valid(P)) return 1;
  float* A4 = cp_prepass(P);
  for (int64_t q = 0; q < n; ++q) {
    tout o; tout_init(&o);
    cp_thread(P, A4, tids[q], 0, exact, NULL, 0, NULL, &o, NULL, 0);
    for (int w = 0; w < o.nw; ++w) { idx[q * P->unroll + w] = o.widx[w]; val[q * P->unroll + w] = o.wval[w]; }
  }
  free(A4);
  return 0;
}
ORA_EXPORT int ora_mriq_threads_out(const ora_mriq_args* P, int32_t exact, const int64_t* tids, int64_t n, float* qr, float* qi) {
  float* KV = mriq_phimag(P);
  for (int64_t q = 0; q < n; ++q) {
    tout o; tout_init(&o);
    mriq_thread(P, KV, tids[q], 0, exact, NULL, 0, NULL, &o, NULL, 0);
    qr[q] = o.wval[0]; qi[q] = o.wval[1];
  }
  free(KV);
  return 0;
}

ORA_EXPORT int64_t ora_tpacf_trips(const ora_tpacf_args* P, int64_t g) { return tp_trips(P, g); }
ORA_EXPORT int64_t ora_tpacf_threads(const ora_tpacf_args* P) { return tp_threads(P); }
ORA_EXPORT int64_t ora_cp_threads(const ora_cp_args* P) { return cp_threads(P); }

/* ------------------------------------------------------------------------------------------ */
/* Plain double-precision definitions (the pins' counterpart: closed forms are tested in       */
/* Python against these and against the FP32 spec sequence).                                   */
/* ------------------------------------------------------------------------------------------ */
ORA_EXPORT void ora_cp_reference_f64(const ora_cp_args* P, double* out, double* mass) {
  for (int y = 0; y < P->ny; ++y)
    for (int x = 0; x < P->nx; ++x) {
      double px = (double)P->h * x, py = (double)P->h * y, s = 0.0, m = 0.0;
      for (int a = 0; a < P->n_atoms; ++a) {
        double dx = px - P->atoms[4 * a], dy = py - P->atoms[4 * a + 1], dz = (double)P->atoms[4 * a + 2] - P->z0;
        double term = P->atoms[4 * a + 3] / sqrt(dx * dx + dy * dy + dz * dz);
        s += term; m += fabs(term);
      }
      out[(size_t)y * P->nx + x] = s;
      if (mass) mass[(size_t)y * P->nx + x] = m;
    }
}

ORA_EXPORT void ora_mriq_reference_f64(const ora_mriq_args* P, double* qr, double* qi, double* mass) {
  const double tp = 2.0 * 3.14159265358979323846;
  for (int v = 0; v < P->n_vox; ++v) {
    double sr = 0, si = 0, m = 0;
    for (int k = 0; k < P->n_k; ++k) {
      double pm = (double)P->phi_r[k] * P->phi_r[k] + (double)P->phi_i[k] * P->phi_i[k];
      double arg = tp * ((double)P->kx[k] * P->x[v] + (double)P->ky[k] * P->y[v] + (double)P->kz[k] * P->z[v]);
      sr += pm * cos(arg); si += pm * sin(arg); m += pm;
    }
    qr[v] = sr; qi[v] = si;
    if (mass) mass[v] = m;
  }
}

/* ------------------------------------------------------------------------------------------ */
/* Value-range profiler (readings R8, R9).                                   */
/* ------------------------------------------------------------------------------------------ */
static float pow10f_table(int k) {
  char buf[16];
  /* T_k = the binary32 value nearest 10^k (decimal literal "1e<k>" parsed as float) */
  int n = 0;
  buf[n++] = '1'; buf[n++] = 'e';
  if (k < 0) { buf[n++] = '-'; k = -k; }
  if (k >= 10) buf[n++] = (char)('0' + k / 10);
  buf[n++] = (char)('0' + k % 10);
  buf[n] = 0;
  return strtof(buf, NULL);
}
ORA_EXPORT float ora_threshold(int32_t k) { return pow10f_table(k); }

/* ranges at threshold T: classes neg (v < -T), zero (-T <= v <= T), pos (v > T). */
static int64_t ranges_at(const float* v, const uint8_t* valid, int64_t n, float T, ora_rset* out) {
  float mn[3], mx[3]; int have[3] = {0, 0, 0};
  for (int64_t s = 0; s < n; ++s) {
    if (valid && !valid[s]) continue;
    float x = v[s];
    int c = (x < -T) ? 0 : (x > T ? 2 : 1);
    if (!have[c]) { mn[c] = mx[c] = x; have[c] = 1; }
    else { if (x < mn[c]) mn[c] = x; if (x > mx[c]) mx[c] = x; }
  }
  int64_t cost = 0; int r = 0;
  for (int c = 0; c < 3; ++c) if (have[c]) {
    cost += ora_ord(mx[c]) - ora_ord(mn[c]) + 1;
    if (out) { out->lo[r] = mn[c]; out->hi[r] = mx[c]; }
    r++;
  }
  if (out) out->n = r;
  return cost;
}

ORA_EXPORT int64_t ora_profile_cost(const float* v, const uint8_t* valid, int64_t n, int32_t k) {
  return ranges_at(v, valid, n, pow10f_table(k), NULL);
}

/* Returns 0, or 6 (HK_ERR_PROFILE_NAN) if a valid sample is NaN/Inf. */
ORA_EXPORT int ora_profile(const float* v, const uint8_t* valid, int64_t n, int32_t t0_exp10, ora_rset* out) {
  memset(out, 0, sizeof(*out));
  int64_t nvalid = 0;
  for (int64_t s = 0; s < n; ++s) {
    if (valid && !valid[s]) continue;
    if (!isfinite(v[s])) return 6;
    nvalid++;
  }
  int k = t0_exp10;
  out->t_exp10 = k;
  if (nvalid == 0) return 0;
  for (;;) {
    int64_t c0 = ora_profile_cost(v, valid, n, k);
    int64_t cm = (k - 1 >= -38) ? ora_profile_cost(v, valid, n, k - 1) : INT64_MAX;
    int64_t cp = (k + 1 <= 38) ? ora_profile_cost(v, valid, n, k + 1) : INT64_MAX;
    if (!(cp < c0 || cm < c0)) break;
    k = (cp <= cm) ? k + 1 : k - 1;
  }
  ranges_at(v, valid, n, pow10f_table(k), out);
  out->t_exp10 = k;
  return 0;
}

/* ------------------------------------------------------------------------------------------ */
/* Output correctness rules (R3-R6) and the 5 classes (L2377-2387).  */
/* ------------------------------------------------------------------------------------------ */
/* err/tol for one element; wrong iff !(err <= tol).  M = max |golden| over the whole output. */
static int fp_elem_wrong(float r, float g, float M, float* ratio) {
  float err = fabsf(r - g);
  float tol = fmaxf(1e-4f * M, 0.002f * fabsf(g));
  float q = err / tol;
  *ratio = isnan(q) ? INFINITY : q;
  return !(err <= tol);
}
ORA_EXPORT int ora_fp_wrong(const float* r, const float* g, int64_t n, float M, float* worst) {
  int wrong = 0; float w = 0.0f;
  for (int64_t e = 0; e < n; ++e) {
    float q;
    if (fp_elem_wrong(r[e], g[e], M, &q)) wrong = 1;
    if (q > w) w = q;
  }
  if (worst) *worst = w;
  return wrong;
}
ORA_EXPORT float ora_max_abs(const float* g, int64_t n) {
  float m = 0.0f;
  for (int64_t e = 0; e < n; ++e) if (fabsf(g[e]) > m) m = fabsf(g[e]);
  return m;
}
/* TPACF outputs (R4): DD[1..nb], DRS[1..nb] = sum_s DR_s, RRS[1..nb] = sum_s RR_s. */
ORA_EXPORT void ora_tpacf_outputs(const int64_t* hist, int32_t n_rand, int32_t n_bins, int64_t* out3nb) {
  int nb2 = n_bins + 2;
  for (int b = 1; b <= n_bins; ++b) {
    int64_t dd = hist[b], rr = 0, dr = 0;
    for (int s = 1; s <= n_rand; ++s) { rr += hist[(int64_t)s * nb2 + b]; dr += hist[(int64_t)(n_rand + s) * nb2 + b]; }
    out3nb[b - 1] = dd; out3nb[n_bins + b - 1] = dr; out3nb[2 * n_bins + b - 1] = rr;
  }
}
/* R3: element wrong iff 100*|h - g| > g, exact integers. */
ORA_EXPORT int ora_tpacf_wrong(const int64_t* hist, const int64_t* golden, int32_t n_rand, int32_t n_bins, float* worst) {
  int64_t a[96], b[96];
  ora_tpacf_outputs(hist, n_rand, n_bins, a);
  ora_tpacf_outputs(golden, n_rand, n_bins, b);
  int wrong = 0; float w = 0.0f;
  for (int e = 0; e < 3 * n_bins; ++e) {
    int64_t d = a[e] - b[e]; if (d < 0) d = -d;
    if (100 * d > b[e]) wrong = 1;
    float q = b[e] > 0 ? (float)(100.0 * (double)d / (double)b[e]) : (d > 0 ? INFINITY : 0.0f);
    if (q > w) w = q;
  }
  if (worst) *worst = w;
  return wrong;
}
/* R1 precedence: failure; else (wrong, alarm) -> 4 classes. */
ORA_EXPORT int32_t ora_classify(int32_t wrong, uint32_t alarm, uint32_t fail) {
  if (fail) return C_FAILURE;
  if (!wrong) return alarm ? C_DET_MASKED : C_MASKED;
  return alarm ? C_DETECTED : C_UNDETECTED;
}

/* ------------------------------------------------------------------------------------------ */
/* Site catalogue and injection decode (R13-R15).                                              */
/* ------------------------------------------------------------------------------------------ */
ORA_EXPORT int32_t ora_nsites(int32_t bench, int32_t unroll) {
  return bench == B_CP ? cp_nsites(unroll) : bench == B_MRIQ ? MRIQ_NSITES : TPACF_NSITES;
}
/* class: SC_NL (one instance per thread) or SC_ITER (golden-trip instances); width 32 or 64 */
ORA_EXPORT void ora_site_info(int32_t bench, int32_t unroll, int32_t site, int32_t* cls, int32_t* width) {
  *cls = SC_ITER; *width = 32;
  if (bench == B_CP) {
    if (site <= 5) *cls = SC_NL;
    if (site == 12 || site == 13) *width = 64;
  } else if (bench == B_MRIQ) {
    if (site <= 3 || site >= MRIQ_PHIMAG_SITE0) *cls = SC_NL;
    if (site >= 9 && site <= 14) *width = 64;
  } else {
    if (site <= 10) *cls = SC_NL;
    if (site == 19 || site == 20) *width = 64;
  }
  (void)unroll;
}

/* Sites that exist only because of HAUBERK (the loop detector's counter / accumulator and the
 * expected trip count): absent from the original program, so the FI-only binary (row a7,
 * "binary with HAUBERK FI ... error sensitivity of baseline program") has none.
 * CP: it (last site); MRI-Q: it (28); TPACF: expect @def (6), expect @live (13), acc (28), cnt (29). */
ORA_EXPORT int32_t ora_detector_site(int32_t bench, int32_t unroll, int32_t site) {
  if (bench == B_CP) return site == cp_nsites(unroll) - 1;
  if (bench == B_MRIQ) return site == 28;
  return site == 6 || site == 13 || site == 28 || site == 29;
}

typedef struct {
  int bench;
  const ora_cp_args* cp; const ora_mriq_args* mq; const ora_tpacf_args* tp;
  int nsites; int nen; int en[64];
  int64_t nthr; int64_t trips_uniform; /* CP / MRI-Q */
  int64_t* prefix; int64_t total_trips;   /* TPACF: prefix[g] = sum of trips of threads < g */
} catalog;

/* Threads of an NL site: PhiMag sites of MRI-Q run on the n_k PhiMag threads. */
static int64_t cat_nl_threads(const catalog* K, int s) {
  if (K->bench == B_MRIQ && s >= MRIQ_PHIMAG_SITE0) return K->mq->n_k;
  return K->nthr;
}

/* variant 0 = FI&FT catalogue; 1 = FI-only (the original program's sites only). */
static void cat_build(catalog* K, int bench, const void* args, uint64_t site_mask, int variant) {
  memset(K, 0, sizeof(*K));
  K->bench = bench;
  int U = 1;
  if (bench == B_CP) { K->cp = (const ora_cp_args*)args; U = K->cp->unroll; K->nthr = cp_threads(K->cp); K->trips_uniform = K->cp->n_atoms; K->total_trips = K->nthr * K->trips_uniform; }
  else if (bench == B_MRIQ) { K->mq = (const ora_mriq_args*)args; K->nthr = K->mq->n_vox; K->trips_uniform = K->mq->n_k; K->total_trips = K->nthr * K->trips_uniform; }
  else {
    K->tp = (const ora_tpacf_args*)args; K->nthr = tp_threads(K->tp);
    K->prefix = (int64_t*)malloc(sizeof(int64_t) * (size_t)(K->nthr + 1));
    K->prefix[0] = 0;
    for (int64_t g = 0; g < K->nthr; ++g) K->prefix[g + 1] = K->prefix[g] + tp_trips(K->tp, g);
    K->total_trips = K->prefix[K->nthr];
  }
  K->nsites = ora_nsites(bench, U);
  for (int s = 0; s < K->nsites; ++s) {
    if (!((site_mask >> s) & 1)) continue;
    if (variant == 1 && ora_detector_site(bench, U, s)) continue;
    int32_t cls, w; ora_site_info(bench, U, s, &cls, &w);
    int64_t D = cls == SC_NL ? cat_nl_threads(K, s) : K->total_trips;
    if (D > 0) K->en[K->nen++] = s;
  }
}
static void cat_free(catalog* K) { free(K->prefix); K->prefix = NULL; }

/* Decode injection n of a campaign over catalogue K: site, (thread, instance), bits (R14-R15).
 * nbits <= 1: one bit = bounded(r_3, width).  nbits = k > 1 (NEXT f1; Fig. 14
 * L2691): k distinct bits by a partial Fisher-Yates shuffle of [0, width): step 0 draws with r_3
 * (so bit 0 equals the single-bit draw), step t >= 1 with output 16n + t of the stream seeded
 * seed ^ 0xD1B54A32D192ED03. */
static void cat_decode(const catalog* K, uint64_t seed, int64_t n, int nbits, ora_fault* f) {
  uint64_t r1 = ora_splitmix(seed, 8 * (uint64_t)n + 1);
  uint64_t r2 = ora_splitmix(seed, 8 * (uint64_t)n + 2);
  uint64_t r3 = ora_splitmix(seed, 8 * (uint64_t)n + 3);
  int s = K->en[ora_bounded(r1, (uint64_t)K->nen)];
  int U = K->cp ? K->cp->unroll : 1;
  int32_t cls, w; ora_site_info(K->bench, U, s, &cls, &w);
  f->site = s; f->hang = 0;
  if (cls == SC_NL) {
    f->thread = (int64_t)ora_bounded(r2, (uint64_t)cat_nl_threads(K, s));
    f->inst = 0;
  } else {
    int64_t u = (int64_t)ora_bounded(r2, (uint64_t)K->total_trips);
    if (!K->prefix) { f->thread = u / K->trips_uniform; f->inst = u % K->trips_uniform; }
    else {
      /* largest g with prefix[g] <= u (binary search over the plain prefix array) */
      int64_t lo = 0, hi = K->nthr; /* invariant: prefix[lo] <= u < prefix[hi] */
      while (hi - lo > 1) { int64_t mid = lo + (hi - lo) / 2; if (K->prefix[mid] <= u) lo = mid; else hi = mid; }
      f->thread = lo; f->inst = u - K->prefix[lo];
    }
  }
  if (nbits <= 1) { f->mask = 1ull << ora_bounded(r3, (uint64_t)w); return; }
  if (nbits > w) nbits = w;
  int perm[64];
  for (int b = 0; b < w; ++b) perm[b] = b;
  uint64_t mask = 0;
  for (int t = 0; t < nbits; ++t) {
    uint64_t r = t == 0 ? r3 : ora_splitmix(seed ^ 0xD1B54A32D192ED03ull, 16 * (uint64_t)n + (uint64_t)t);
    int j = t + (int)ora_bounded(r, (uint64_t)(w - t));
    int tmp = perm[t]; perm[t] = perm[j]; perm[j] = tmp;
    mask |= 1ull << perm[t];
  }
  f->mask = mask;
}

/* Public decode: bench_mode >= 0 fixes the benchmark, -1 = mixed (bench = n mod 3). */
ORA_EXPORT int ora_decode(int32_t bench_mode, const void* const args[3], const uint64_t site_mask[3],
                          uint64_t seed, int32_t nbits, int32_t variant, int64_t first, int64_t count,
                          int32_t* bench_out, ora_fault* out) {
  catalog K[3]; int have[3] = {0, 0, 0};
  for (int64_t q = 0; q < count; ++q) {
    int64_t n = first + q;
    int b = bench_mode >= 0 ? bench_mode : (int)(n % 3);
    if (!have[b]) { cat_build(&K[b], b, args[b], site_mask[b], variant); have[b] = 1; if (K[b].nen == 0) return 1; }
    bench_out[q] = b;
    cat_decode(&K[b], seed, n, nbits, &out[q]);
  }
  for (int b = 0; b < 3; ++b) if (have[b]) cat_free(&K[b]);
  return 0;
}

/* ------------------------------------------------------------------------------------------ */
/* Campaign: golden run, then one classified experiment per injection.      */
/* mode 0 = replica (every thread re-run, the faithful definition);                            */
/* mode 1 = replay (only the faulted thread; golden patched — R22; equal to replica by the     */
/*          additive-write semantics R18, checked by tests on small shapes).                    */
/* ------------------------------------------------------------------------------------------ */
typedef struct {
  float* g0; float* g1; int64_t* gh; float M; /* golden outputs, max |golden| */
  float* A4; float* KV;
} goldens;

static int golden_build(int b, const void* args, int exact, int vf, const ora_ranges* R, goldens* G) {
  memset(G, 0, sizeof(*G));
  ora_runinfo I;
  if (b == B_CP) {
    const ora_cp_args* P = (const ora_cp_args*)args;
    G->g0 = (float*)malloc(sizeof(float) * (size_t)P->nx * P->ny);
    if (ora_cp_run(P, vf, exact, R, R->n_det, NULL, G->g0, NULL, &I)) return 1;
    G->M = ora_max_abs(G->g0, (int64_t)P->nx * P->ny);
    G->A4 = cp_prepass(P);
  } else if (b == B_MRIQ) {
    const ora_mriq_args* P = (const ora_mriq_args*)args;
    G->g0 = (float*)malloc(sizeof(float) * (size_t)(P->n_vox > 0 ? P->n_vox : 1) * 2);
    G->g1 = G->g0 + P->n_vox;
    if (ora_mriq_run(P, vf, exact, R, R->n_det, NULL, G->g0, G->g1, NULL, &I)) return 1;
    G->M = ora_max_abs(G->g0, 2LL * P->n_vox); /* R6: max over [Qr; Qi] */
    G->KV = mriq_phimag(P);
  } else {
    const ora_tpacf_args* P = (const ora_tpacf_args*)args;
    G->gh = (int64_t*)malloc(sizeof(int64_t) * (size_t)tp_nh(P) * (P->n_bins + 2));
    if (ora_tpacf_run(P, vf, R, R->n_det, NULL, G->gh, NULL, &I)) return 1;
  }
  return I.alarm != 0 ? 2 : 0; /* fault-free run must not alarm (train = test, L2402-2403) */
}
static void golden_free(goldens* G) { free(G->g0); free(G->gh); free(G->A4); free(G->KV); }

/* Replay one injection; fills the record's wrong/alarm/fail/domain/margin/worst. */
static void replay_one(int b, const void* args, int exact, int vf, const ora_ranges* R, const goldens* G,
                       const ora_fault* f, ora_record* rec, int32_t* wrong_out) {
  fctx F = {1, f->site, f->inst, f->mask, 0, f->hang > 0 ? f->hang : 10};
  tout o; tout_init(&o);
  int wrong = 0; float worst = 0.0f;
  if (b == B_CP || b == B_MRIQ) {
    /* own elements (the golden twin's writes) are removed; faulted writes are added (R18) */
    int64_t own_idx[16]; int32_t own_buf[16]; int nown = 0;
    if (b == B_CP) {
      const ora_cp_args* P = (const ora_cp_args*)args;
      tout g; tout_init(&g);
      cp_thread(P, G->A4, f->thread, vf, exact, R, R->n_det, NULL, &g, NULL, 0);
      for (int w = 0; w < g.nw; ++w) { own_idx[nown] = g.widx[w]; own_buf[nown] = 0; nown++; }
      cp_thread(P, G->A4, f->thread, vf | F_FI, exact, R, R->n_det, &F, &o, NULL, 0);
    } else {
      const ora_mriq_args* P = (const ora_mriq_args*)args;
      tout g; tout_init(&g);
      mriq_thread(P, G->KV, f->thread, vf, exact, R, R->n_det, NULL, &g, NULL, 0);
      for (int w = 0; w < g.nw; ++w) { own_idx[nown] = g.widx[w]; own_buf[nown] = g.wbuf[w]; nown++; }
      mriq_thread(P, G->KV, f->thread, vf | F_FI, exact, R, R->n_det, &F, &o, NULL, 0);
    }
    if (!o.fail) {
      /* touched = own ∪ written; new value = (own ? 0 : golden) + sum of faulted writes */
      int64_t tidx[32]; int32_t tbuf[32]; int nt = 0;
      for (int a = 0; a < nown; ++a) { tidx[nt] = own_idx[a]; tbuf[nt] = own_buf[a]; nt++; }
      for (int w = 0; w < o.nw; ++w) {
        int dup = 0;
        for (int a = 0; a < nt; ++a) if (tidx[a] == o.widx[w] && tbuf[a] == o.wbuf[w]) dup = 1;
        if (!dup) { tidx[nt] = o.widx[w]; tbuf[nt] = o.wbuf[w]; nt++; }
      }
      for (int a = 0; a < nt; ++a) {
        const float* gb = tbuf[a] ? G->g1 : G->g0;
        int own = 0;
        for (int q = 0; q < nown; ++q) if (own_idx[q] == tidx[a] && own_buf[q] == tbuf[a]) own = 1;
        float v = own ? 0.0f : gb[tidx[a]];
        for (int w = 0; w < o.nw; ++w) if (o.widx[w] == tidx[a] && o.wbuf[w] == tbuf[a]) v = v + o.wval[w];
        float q;
        if (fp_elem_wrong(v, gb[tidx[a]], G->M, &q)) wrong = 1;
        if (q > worst) worst = q;
      }
    }
  } else {
    const ora_tpacf_args* P = (const ora_tpacf_args*)args;
    size_t nh = (size_t)tp_nh(P) * (P->n_bins + 2);
    int64_t* hist = (int64_t*)malloc(sizeof(int64_t) * nh);
    memcpy(hist, G->gh, sizeof(int64_t) * nh);
    int64_t* d = (int64_t*)calloc(nh, sizeof(int64_t));
    tout g; tout_init(&g);
    tpacf_thread(P, f->thread, vf, R, R->n_det, NULL, &g, d, NULL, 0);
    for (size_t e = 0; e < nh; ++e) { hist[e] -= d[e]; d[e] = 0; }
    tpacf_thread(P, f->thread, vf | F_FI, R, R->n_det, &F, &o, d, NULL, 0);
    for (size_t e = 0; e < nh; ++e) hist[e] += d[e];
    if (!o.fail) wrong = ora_tpacf_wrong(hist, G->gh, P->n_rand, P->n_bins, &worst);
    free(hist); free(d);
  }
  rec->alarm = o.alarm; rec->fail = o.fail; rec->domain = o.domain; rec->margin = o.margin; rec->gap = o.gap;
  rec->worst = worst;
  *wrong_out = wrong;
}

static void replica_one(int b, const void* args, int exact, int vf, const ora_ranges* R, const goldens* G,
                        const ora_fault* f, ora_record* rec, int32_t* wrong_out) {
  ora_runinfo I; int wrong = 0; float worst = 0.0f;
  if (b == B_CP) {
    const ora_cp_args* P = (const ora_cp_args*)args;
    int64_t n = (int64_t)P->nx * P->ny;
    float* out = (float*)malloc(sizeof(float) * (size_t)n);
    ora_cp_run(P, vf, exact, R, R->n_det, f, out, NULL, &I);
    if (!I.fail) wrong = ora_fp_wrong(out, G->g0, n, G->M, &worst);
    free(out);
  } else if (b == B_MRIQ) {
    const ora_mriq_args* P = (const ora_mriq_args*)args;
    float* out = (float*)malloc(sizeof(float) * 2 * (size_t)(P->n_vox > 0 ? P->n_vox : 1));
    ora_mriq_run(P, vf, exact, R, R->n_det, f, out, out + P->n_vox, NULL, &I);
    if (!I.fail) wrong = ora_fp_wrong(out, G->g0, 2LL * P->n_vox, G->M, &worst);
    free(out);
  } else {
    const ora_tpacf_args* P = (const ora_tpacf_args*)args;
    int64_t* hist = (int64_t*)malloc(sizeof(int64_t) * (size_t)tp_nh(P) * (P->n_bins + 2));
    ora_tpacf_run(P, vf, R, R->n_det, f, hist, NULL, &I);
    if (!I.fail) wrong = ora_tpacf_wrong(hist, G->gh, P->n_rand, P->n_bins, &worst);
    free(hist);
  }
  rec->alarm = I.alarm; rec->fail = I.fail; rec->domain = I.domain; rec->margin = I.margin; rec->gap = I.gap;
  rec->worst = worst;
  *wrong_out = wrong;
}

/* counts[b*5 + cls] += 1 for each injection; records (nullable) get one entry per injection. */
/* variant 0 = FI&FT binary (HAUBERK-NL + HAUBERK-L); 1 = FI-only binary (the original program with
 * the injector: its catalogue holds the original program's sites only, its
 * outcomes are masked / undetected (SDC) / failure).  hang_factor = R17's T (0 -> 10). */
ORA_EXPORT int ora_campaign(int32_t bench_mode, const void* const args[3], const ora_ranges* const ranges[3],
                            const uint64_t site_mask[3], uint64_t seed, int32_t nbits, int64_t first, int64_t count,
                            int32_t exact, int32_t mode, int32_t variant, int32_t hang_factor,
                            ora_record* records, int64_t* counts) {
  catalog K[3]; goldens G[3]; int have[3] = {0, 0, 0};
  const int vf = variant == 1 ? 0 : (F_NL | F_L);
  int rc = 0;
  for (int64_t q = 0; q < count && rc == 0; ++q) {
    int64_t n = first + q;
    int b = bench_mode >= 0 ? bench_mode : (int)(n % 3);
    if (!have[b]) {
      have[b] = 1;
      cat_build(&K[b], b, args[b], site_mask[b], variant);
      if (K[b].nen == 0) { rc = 1; break; }
      rc = golden_build(b, args[b], exact, vf, ranges[b], &G[b]);
      if (rc) break;
    }
    ora_fault f; cat_decode(&K[b], seed, n, nbits, &f);
    f.hang = hang_factor;
    ora_record rec; memset(&rec, 0, sizeof(rec));
    int32_t wrong = 0;
    /* replay cannot express a PhiMag fault (it reaches every voxel, R22): run that one as a replica */
    if (mode == 1 && !(b == B_MRIQ && f.site >= MRIQ_PHIMAG_SITE0)) replay_one(b, args[b], exact, vf, ranges[b], &G[b], &f, &rec, &wrong);
    else replica_one(b, args[b], exact, vf, ranges[b], &G[b], &f, &rec, &wrong);
    rec.index = n; rec.bench = b; rec.site = f.site; rec.thread = f.thread; rec.inst = f.inst; rec.mask = f.mask;
    rec.cls = ora_classify(wrong, rec.alarm, rec.fail);
    if (records) records[q] = rec;
    if (counts) counts[b * 5 + rec.cls] += 1;
  }
  for (int b = 0; b < 3; ++b) if (have[b]) { cat_free(&K[b]); golden_free(&G[b]); }
  return rc;
}

/* ------------------------------------------------------------------------------------------ */
/* A6: loop-detector target selection (PAPER L1221-1273 [§V.B step i], Fig. 9).     */
/* The loop's dataflow graph: node kinds A6_VAR (virtual variable defined in the loop), A6_TEMP  */
/* (temporary of a multi-operation statement, L1246-1250), A6_LOAD (memory-load data, counted:   */
/* "including the memory load data", L1253-1254), A6_CONST (not counted: "but not the          */
/* constant"), A6_NLPROT (loop invariants protected by non-loop detectors, excluded L1254-1257),  */
/* A6_ACCOP (the operation of a self-accumulator's own update statement, `E += w * t`: part of   */
/* the target's definition, not of its backward set — the reading under which Fig. 9 gives 12   */
/* and 13, DESIGN R12), A6_IND (the loop's induction variable: protected by the iteration       */
/* counter, L1293-1300, so neither counted nor a candidate).  Edge k: src[k] is used to compute  */
/* dst[k] (a load's address is not data); self-edges (E = E + ...) are ignored.                 */
/* ------------------------------------------------------------------------------------------ */
enum { A6_VAR = 0, A6_TEMP = 1, A6_LOAD = 2, A6_CONST = 3, A6_NLPROT = 4, A6_ACCOP = 5, A6_IND = 6 };

static void a6_ancestors(int32_t n, int32_t ne, const int32_t* src, const int32_t* dst, int32_t v, uint8_t* mark) {
  /* plain iterative closure: mark every u with a path u ->* v (v itself not marked) */
  memset(mark, 0, (size_t)n);
  int changed = 1;
  while (changed) {
    changed = 0;
    for (int32_t k = 0; k < ne; ++k) {
      if (src[k] == dst[k]) continue;
      if ((dst[k] == v || mark[dst[k]]) && !mark[src[k]] && src[k] != v) { mark[src[k]] = 1; changed = 1; }
    }
  }
}

/* Cumulative backward dataflow dependency of v over the nodes not yet `removed` (nullable). */
ORA_EXPORT int32_t ora_a6_count(int32_t n, const int32_t* kind, int32_t ne, const int32_t* src, const int32_t* dst,
                                const uint8_t* removed, int32_t v) {
  uint8_t* mark = (uint8_t*)malloc((size_t)(n > 0 ? n : 1));
  a6_ancestors(n, ne, src, dst, v, mark);
  int32_t c = 0;
  for (int32_t u = 0; u < n; ++u)
    if (mark[u] && !(removed && removed[u]) && (kind[u] == A6_VAR || kind[u] == A6_TEMP || kind[u] == A6_LOAD)) c++;
  free(mark);
  return c;
}

/* Selection repeated Maxvar times (L1259-1273): candidates are the loop's virtual variables not
 * yet removed, self-accumulators first (they need no accumulator code, L1223-1225); the one with
 * the largest cumulative backward dependency wins, ties to the earlier node (program order, R12);
 * the winner and every node with forward dependency to it are then removed.  Returns the number
 * selected; order[0..] = the chosen node ids. */
ORA_EXPORT int32_t ora_a6_select(int32_t n, const int32_t* kind, const uint8_t* selfacc, int32_t ne, const int32_t* src,
                                 const int32_t* dst, int32_t maxvar, int32_t* order) {
  uint8_t* removed = (uint8_t*)calloc((size_t)(n > 0 ? n : 1), 1);
  uint8_t* mark = (uint8_t*)malloc((size_t)(n > 0 ? n : 1));
  int32_t got = 0;
  for (; got < maxvar; ++got) {
    int any_self = 0;
    for (int32_t u = 0; u < n; ++u) if (kind[u] == A6_VAR && !removed[u] && selfacc[u]) any_self = 1;
    int32_t best = -1, bc = -1;
    for (int32_t u = 0; u < n; ++u) {
      if (kind[u] != A6_VAR || removed[u] || (any_self && !selfacc[u])) continue;
      int32_t c = ora_a6_count(n, kind, ne, src, dst, removed, u);
      if (c > bc) { bc = c; best = u; }
    }
    if (best < 0) break;
    order[got] = best;
    a6_ancestors(n, ne, src, dst, best, mark);
    removed[best] = 1;
    for (int32_t u = 0; u < n; ++u) if (mark[u]) removed[u] = 1;
  }
  free(removed); free(mark);
  return got;
}

/* ------------------------------------------------------------------------------------------ */
/* Recovery and evaluation arithmetic (PAPER §VI, §VIII).                */
/* ------------------------------------------------------------------------------------------ */
/* R10/R11 range check of a single value against detector d (alpha applied to the bounds). */
ORA_EXPORT int32_t ora_in_range(const ora_ranges* R, int32_t d, float v) {
  uint32_t m = 0xffffffffu; float g = INFINITY;
  return in_range(R, d, v, &m, &g);
}

/* A11 (L1309-1313: "calculates new ranges that include the outlier"; DESIGN R24): each value joins
 * the range of its correlation class at the detector's threshold T = 10^t_exp10 (neg: v < -T,
 * zero: -T <= v <= T, pos: v > T); a class without a range gains one.  Ranges stay in class order.
 * Non-finite values are ignored (they cannot be represented by a range).  Returns ranges added. */
ORA_EXPORT int32_t ora_extend_ranges(ora_rset* s, const float* values, int32_t nv) {
  const float T = pow10f_table(s->t_exp10);
  float lo[3], hi[3]; int have[3] = {0, 0, 0};
  for (int r = 0; r < s->n; ++r) {
    float x = s->lo[r];
    int c = (x < -T) ? 0 : (x > T ? 2 : 1);
    lo[c] = s->lo[r]; hi[c] = s->hi[r]; have[c] = 1;
  }
  int before = s->n, added = 0;
  for (int32_t k = 0; k < nv; ++k) {
    float x = values[k];
    if (!isfinite(x)) continue;
    int c = (x < -T) ? 0 : (x > T ? 2 : 1);
    if (!have[c]) { lo[c] = hi[c] = x; have[c] = 1; added++; }
    else { if (x < lo[c]) lo[c] = x; if (x > hi[c]) hi[c] = x; }
  }
  int r = 0;
  for (int c = 0; c < 3; ++c) if (have[c]) { s->lo[r] = lo[c]; s->hi[r] = hi[c]; r++; }
  s->n = r;
  (void)before;
  return added;
}

/* alpha controller (L2066-2077): false-positive ratio above `hi` (10 %) -> alpha x 10; below `lo`
 * (5 %) -> alpha / 10 while alpha stays >= 1 (i.e. only from alpha >= 10). */
ORA_EXPORT float ora_alpha_step(float alpha, double fp_ratio, double hi, double lo) {
  if (fp_ratio > hi) return alpha * 10.0f;
  if (fp_ratio < lo && alpha >= 10.0f) return alpha / 10.0f;
  return alpha;
}

/* Re-execution diagnosis (Fig. 11).  0 ok (no alarm), 1 false alarm (re-run alarms
 * again with a bitwise-identical output), 2 transient (re-run ends normally without an alarm: its
 * output is taken), 3 persistent (re-run alarms with a different output: BIST / migration), 4 failure
 * (either run crashed or hung: the guardian's path, L1982-2007). */
ORA_EXPORT int32_t ora_diagnose(uint32_t alarm1, uint32_t fail1, uint32_t alarm2, uint32_t fail2, int32_t identical) {
  if (fail1) return 4;
  if (!alarm1) return 0;
  if (fail2) return 4;
  if (!alarm2) return 2;
  return identical ? 1 : 3;
}

/* Campaign summary (R2, L2372-2375 and L2480-2483: coverage = P(detected or masked), failures
 * covered): out[0] coverage = 1 - undetected/total; out[1] SDC ratio = undetected/total (for an
 * FI-only campaign: the unprotected SDC rate, L211-213); out[2] detected (classes 1+2)/total;
 * out[3] failure/total.  counts: int64 [5] (one benchmark) — sum rows first for several. */
ORA_EXPORT int32_t ora_coverage(const int64_t* counts5, double* out4) {
  int64_t tot = 0;
  for (int c = 0; c < 5; ++c) tot += counts5[c];
  if (tot == 0) { for (int k = 0; k < 4; ++k) out4[k] = NAN; return 1; }
  out4[0] = 1.0 - (double)counts5[C_UNDETECTED] / (double)tot;
  out4[1] = (double)counts5[C_UNDETECTED] / (double)tot;
  out4[2] = (double)(counts5[C_DET_MASKED] + counts5[C_DETECTED]) / (double)tot;
  out4[3] = (double)counts5[C_FAILURE] / (double)tot;
  return 0;
}

ORA_EXPORT int ora_version(void) { return 2; }
