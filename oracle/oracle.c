/*
 * oracle.c -- plain, slow, obviously-correct CPU oracle of one SPH time step.
 *
 * TEST INFRASTRUCTURE ONLY.  Nothing on the product path may link, load or
 * call this file: only tests/, __graft_entry__.smoke() and bench.py's
 * cpu_baseline / --impl reference legs use it.  It shares no code, header,
 * table or constant generator with the CUDA library (libsph); the two meet
 * only through the seeded initial conditions of paper_conf_sc_simsekpc24_b200/ics.py.
 *
 * What it follows.  PAPER.md (Simsek, Piccinali, Ciorba, SC'24 workshops)
 * fixes the *structure* of the step it measures -- a GPU-resident SPH-EXA
 * time step made of DomainDecompAndSync (particle keys), XMass
 * (P:184), IADVelocityDivCurl, MomentumEnergy and an
 * end-of-step collective computing the time step -- but prints no
 * SPH formula.  Every formula below is therefore the reading recorded in
 * SURVEY.md section 8(c) ("Algorithm, step by step", items 1-10) and listed
 * in DESIGN.md section 3; each function names the item it follows.
 *
 * Style rules (so the code can be checked against the text by eye):
 *   - fp64 everywhere, compiled with -O2 -ffp-contract=off (no FMA);
 *   - libm sin/sqrt/pow, IEEE division;
 *   - neighbours by O(N^2) brute force, the definition;
 *   - every sum runs over j in ascending order of the current particle order;
 *   - OpenMP only over the independent target index i.
 *
 * Pins: tests/test_oracle_*.py check every function here against closed
 * forms, golden values (tests/golden/), invariants and library routines.
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#ifndef M_PI
#define M_PI 3.14159265358979323846
#endif

/* Parameters of the step (SURVEY 8(c) "Parameter table"). */
typedef struct {
  double box_min[3];     /* periodic axes: fixed box; open axes: ignored (bbox) */
  double box_max[3];
  int32_t periodic[3];   /* 1 = periodic axis                                    */
  int32_t eos;           /* 0 = ideal gas, 1 = isothermal                        */
  double gamma;          /* ideal-gas adiabatic index                            */
  double cs0;            /* isothermal sound speed                               */
  double K;              /* sinc-kernel normalisation for n = 6                  */
  double ng0;            /* target neighbour count for the h update              */
  double k_cour;         /* Courant factor C                                     */
  double dt_max_growth;  /* dt <= growth * dt_prev                               */
  double av_alpha, av_beta, av_eps;
  double h_cap;          /* h <= h_cap after the update                          */
} oracle_params;

enum { ORACLE_OK = 0, ORACLE_ERR_BOX = 1, ORACLE_ERR_SINGULAR = 2, ORACLE_ERR_CAP = 3 };

/* ---------------------------------------------------------------------------
 * Kernel (SURVEY 8(c) parameter table, "kernel"):
 *   W(r,h) = (K/h^3) * S(pi r / 2h)^6  for r < 2h,   0 for r >= 2h,
 *   S(x) = sin(x)/x,  S(0) = 1.
 * ------------------------------------------------------------------------- */
double oracle_sinc(double x) { return x == 0.0 ? 1.0 : sin(x) / x; }

double oracle_W(double r, double h, double K) {
  if (r >= 2.0 * h) return 0.0;
  double s = oracle_sinc(M_PI * r / (2.0 * h));
  return K / (h * h * h) * pow(s, 6.0);
}

/* dW/dh of the same kernel at fixed r (NormalizationGradh, DESIGN.md reading
 * 21).  With x = pi r / 2h, dx/dh = -x/h and x S'(x) = cos x - S(x):
 *   dW/dh = -(K/h^4) S(x)^5 (6 cos x - 3 S(x))  for r < 2h,  0 for r >= 2h
 * (at r = 0: -3K/h^4 = d/dh of K/h^3). */
double oracle_dWdh(double r, double h, double K) {
  if (r >= 2.0 * h) return 0.0;
  double x = M_PI * r / (2.0 * h);
  double s = oracle_sinc(x);
  return -K / (h * h * h * h) * pow(s, 5.0) * (6.0 * cos(x) - 3.0 * s);
}

/* Minimum image of one coordinate difference:
 * raw difference first, then one conditional +-L. */
static double min_image(double dx, double L, int periodic) {
  if (periodic) {
    if (dx > 0.5 * L) dx -= L;
    else if (dx < -0.5 * L) dx += L;
  }
  return dx;
}

/* d = x_i - x_j (minimum image) and d2 = (dx*dx + dy*dy) + dz*dz, each
 * operation rounded separately (no FMA: -ffp-contract=off). */
static double pair_d(const double* x, const double* y, const double* z, int64_t i, int64_t j,
                     const double* bmin, const double* bmax, const int32_t* per, double d[3]) {
  d[0] = min_image(x[i] - x[j], bmax[0] - bmin[0], per[0]);
  d[1] = min_image(y[i] - y[j], bmax[1] - bmin[1], per[1]);
  d[2] = min_image(z[i] - z[j], bmax[2] - bmin[2], per[2]);
  return (d[0] * d[0] + d[1] * d[1]) + d[2] * d[2];
}

/* ---------------------------------------------------------------------------
 * Step 1, box.  Periodic axes are fixed; open axes take [min_i x, max_i x].
 * ------------------------------------------------------------------------- */
int oracle_box(int64_t n, const double* x, const double* y, const double* z,
               const oracle_params* P, double bmin[3], double bmax[3]) {
  const double* c[3] = {x, y, z};
  for (int a = 0; a < 3; ++a) {
    if (P->periodic[a]) {
      bmin[a] = P->box_min[a];
      bmax[a] = P->box_max[a];
      continue;
    }
    if (n < 1) return ORACLE_ERR_BOX;
    double lo = c[a][0], hi = c[a][0];
    for (int64_t i = 1; i < n; ++i) {
      if (c[a][i] < lo) lo = c[a][i];
      if (c[a][i] > hi) hi = c[a][i];
    }
    if (!(hi > lo)) return ORACLE_ERR_BOX;
    bmin[a] = lo;
    bmax[a] = hi;
  }
  return ORACLE_OK;
}

/* ---------------------------------------------------------------------------
 * Step 2, keys.  s = (x - xmin)/L; ix = min(floor(s * 2^21), 2^21 - 1),
 * clamped at 0; key = sum_b bit_b(ix)<<(3b+2) | bit_b(iy)<<(3b+1) | bit_b(iz)<<3b.
 * ------------------------------------------------------------------------- */
static uint64_t coord21(double v, double lo, double hi) {
  double s = (v - lo) / (hi - lo);
  double f = floor(s * 2097152.0);
  if (f < 0.0) f = 0.0;
  if (f > 2097151.0) f = 2097151.0;
  return (uint64_t)f;
}

uint64_t oracle_morton(uint64_t ix, uint64_t iy, uint64_t iz) {
  uint64_t key = 0;
  for (int b = 0; b < 21; ++b) {
    key |= ((ix >> b) & 1u) << (3 * b + 2);
    key |= ((iy >> b) & 1u) << (3 * b + 1);
    key |= ((iz >> b) & 1u) << (3 * b);
  }
  return key;
}

void oracle_keys(int64_t n, const double* x, const double* y, const double* z,
                 const double bmin[3], const double bmax[3], uint64_t* keys) {
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < n; ++i)
    keys[i] = oracle_morton(coord21(x[i], bmin[0], bmax[0]), coord21(y[i], bmin[1], bmax[1]),
                            coord21(z[i], bmin[2], bmax[2]));
}

/* ---------------------------------------------------------------------------
 * Step 3, sort.  Stable sort of the current order by key: ties keep the
 * current order.  Written as a sort on the pair (key, current index), which
 * is the same total order.  perm[k] = current index of the k-th particle.
 * ------------------------------------------------------------------------- */
typedef struct { uint64_t key; int64_t idx; } key_idx;

static int cmp_key_idx(const void* a, const void* b) {
  const key_idx* p = (const key_idx*)a;
  const key_idx* q = (const key_idx*)b;
  if (p->key != q->key) return p->key < q->key ? -1 : 1;
  if (p->idx != q->idx) return p->idx < q->idx ? -1 : 1;
  return 0;
}

void oracle_sort_order(int64_t n, const uint64_t* keys, int64_t* perm) {
  key_idx* t = (key_idx*)malloc(sizeof(key_idx) * (size_t)(n > 0 ? n : 1));
  for (int64_t i = 0; i < n; ++i) { t[i].key = keys[i]; t[i].idx = i; }
  qsort(t, (size_t)n, sizeof(key_idx), cmp_key_idx);
  for (int64_t i = 0; i < n; ++i) perm[i] = t[i].idx;
  free(t);
}

/* ---------------------------------------------------------------------------
 * Step 4, neighbours.  j in N(i) iff j != i and d2_ij < (2 h_i)*(2 h_i).
 * Brute force over all j, ascending.  Two calls: counts, then lists (CSR,
 * offsets[n+1] precomputed by the caller from the counts).
 * ------------------------------------------------------------------------- */
void oracle_neighbor_counts(int64_t n, const double* x, const double* y, const double* z,
                            const double* h, const double bmin[3], const double bmax[3],
                            const int32_t per[3], int32_t* nc) {
#pragma omp parallel for schedule(dynamic, 16)
  for (int64_t i = 0; i < n; ++i) {
    double d[3], r2max = (2.0 * h[i]) * (2.0 * h[i]);
    int32_t c = 0;
    for (int64_t j = 0; j < n; ++j)
      if (j != i && pair_d(x, y, z, i, j, bmin, bmax, per, d) < r2max) ++c;
    nc[i] = c;
  }
}

void oracle_neighbor_lists(int64_t n, const double* x, const double* y, const double* z,
                           const double* h, const double bmin[3], const double bmax[3],
                           const int32_t per[3], const int64_t* offsets, int64_t* idx) {
#pragma omp parallel for schedule(dynamic, 16)
  for (int64_t i = 0; i < n; ++i) {
    double d[3], r2max = (2.0 * h[i]) * (2.0 * h[i]);
    int64_t o = offsets[i];
    for (int64_t j = 0; j < n; ++j)
      if (j != i && pair_d(x, y, z, i, j, bmin, bmax, per, d) < r2max) idx[o++] = j;
  }
}

/* Particles l with d2(t, l) < R*R (l != t included as well as t itself),
 * ascending; returns how many were found (writes at most cap). */
int64_t oracle_ball(int64_t n, const double* x, const double* y, const double* z, int64_t t,
                    double R, const double bmin[3], const double bmax[3], const int32_t per[3],
                    int64_t* out, int64_t cap) {
  double d[3];
  int64_t c = 0;
  for (int64_t l = 0; l < n; ++l)
    if (pair_d(x, y, z, t, l, bmin, bmax, per, d) < R * R) {
      if (c < cap) out[c] = l;
      ++c;
    }
  return c;
}

/* ---------------------------------------------------------------------------
 * Step 5, density (XMass reading):
 *   rho_i = (K/h_i^3) * [ m_i + sum_{j in N(i)} m_j S(pi r_ij / 2h_i)^6 ],
 *   r = sqrt(d2).  All terms are positive, so the |term| scale is rho itself.
 * ------------------------------------------------------------------------- */
void oracle_density(int64_t n, const double* x, const double* y, const double* z,
                    const double* h, const double* m, const double bmin[3], const double bmax[3],
                    const int32_t per[3], const int64_t* off, const int64_t* idx,
                    const oracle_params* P, double* rho) {
#pragma omp parallel for schedule(dynamic, 64)
  for (int64_t i = 0; i < n; ++i) {
    double d[3], sum = m[i];
    for (int64_t k = off[i]; k < off[i + 1]; ++k) {
      int64_t j = idx[k];
      double r = sqrt(pair_d(x, y, z, i, j, bmin, bmax, per, d));
      sum += m[j] * pow(oracle_sinc(M_PI * r / (2.0 * h[i])), 6.0);
    }
    rho[i] = P->K / (h[i] * h[i] * h[i]) * sum;
  }
}

/* ---------------------------------------------------------------------------
 * NormalizationGradh (reading 21), optional step 5b:
 *   Omega_i = 1 + (h_i / (3 rho_i)) * [ m_i dW/dh(0, h_i)
 *                                       + sum_{j in N(i)} m_j dW/dh(r_ij, h_i) ]
 * i.e. 1 - (dh/drho) drho/dh with h proportional to rho^(-1/3).  The
 * momentum-energy step then uses p/(Omega rho^2) in place of p/rho^2.
 * dsum_abs = m_i |dW/dh(0)| + sum_j m_j |dW/dh| (tolerance scale of the sum).
 * ------------------------------------------------------------------------- */
void oracle_gradh(int64_t n, const double* x, const double* y, const double* z,
                  const double* h, const double* m, const double* rho, const double bmin[3],
                  const double bmax[3], const int32_t per[3], const int64_t* off,
                  const int64_t* idx, const oracle_params* P, double* omega, double* dsum,
                  double* dsum_abs) {
#pragma omp parallel for schedule(dynamic, 64)
  for (int64_t i = 0; i < n; ++i) {
    double d[3];
    double t0 = m[i] * oracle_dWdh(0.0, h[i], P->K);
    double sum = t0, sabs = fabs(t0);
    for (int64_t k = off[i]; k < off[i + 1]; ++k) {
      int64_t j = idx[k];
      double r = sqrt(pair_d(x, y, z, i, j, bmin, bmax, per, d));
      double t = m[j] * oracle_dWdh(r, h[i], P->K);
      sum += t;
      sabs += fabs(t);
    }
    dsum[i] = sum;
    dsum_abs[i] = sabs;
    omega[i] = 1.0 + h[i] / (3.0 * rho[i]) * sum;
  }
}

/* ---------------------------------------------------------------------------
 * Step 6, equation of state.
 *   ideal:      p = (gamma-1) rho u,   c = sqrt(gamma (gamma-1) u)
 *   isothermal: p = c0^2 rho,          c = c0
 * ------------------------------------------------------------------------- */
void oracle_eos(int64_t n, const double* rho, const double* u, const oracle_params* P, double* p,
                double* c) {
  for (int64_t i = 0; i < n; ++i) {
    if (P->eos == 0) {
      p[i] = (P->gamma - 1.0) * rho[i] * u[i];
      c[i] = sqrt(P->gamma * (P->gamma - 1.0) * u[i]);
    } else {
      p[i] = P->cs0 * P->cs0 * rho[i];
      c[i] = P->cs0;
    }
  }
}

/* ---------------------------------------------------------------------------
 * Step 7, IAD matrices (IADVelocityDivCurl, matrix part):
 *   Delta = -d = x_j - x_i (minimum image)
 *   tau_i^{ab} = sum_j (m_j/rho_j) W(r_ij, h_i) Delta^a Delta^b
 *   C_i = tau_i^{-1} by the adjugate; det <= 0 or non-finite -> singular.
 * Storage order of the 6 symmetric entries: 11, 12, 13, 22, 23, 33.
 * tau_abs holds sum_j |term| per entry (the tolerance scale of SURVEY 8(c)).
 * ------------------------------------------------------------------------- */
int oracle_iad(int64_t n, const double* x, const double* y, const double* z, const double* h,
               const double* m, const double* rho, const double bmin[3], const double bmax[3],
               const int32_t per[3], const int64_t* off, const int64_t* idx,
               const oracle_params* P, double* C /* n x 6 */, double* tau /* n x 6 */,
               double* tau_abs /* n x 6 */) {
  int status = ORACLE_OK;
#pragma omp parallel for schedule(dynamic, 64)
  for (int64_t i = 0; i < n; ++i) {
    double t[6] = {0, 0, 0, 0, 0, 0}, ta[6] = {0, 0, 0, 0, 0, 0};
    for (int64_t k = off[i]; k < off[i + 1]; ++k) {
      int64_t j = idx[k];
      double d[3];
      double r = sqrt(pair_d(x, y, z, i, j, bmin, bmax, per, d));
      double D[3] = {-d[0], -d[1], -d[2]};
      double vw = (m[j] / rho[j]) * oracle_W(r, h[i], P->K);
      double term[6] = {vw * D[0] * D[0], vw * D[0] * D[1], vw * D[0] * D[2],
                        vw * D[1] * D[1], vw * D[1] * D[2], vw * D[2] * D[2]};
      for (int e = 0; e < 6; ++e) { t[e] += term[e]; ta[e] += fabs(term[e]); }
    }
    double t11 = t[0], t12 = t[1], t13 = t[2], t22 = t[3], t23 = t[4], t33 = t[5];
    double det = t11 * (t22 * t33 - t23 * t23) - t12 * (t12 * t33 - t23 * t13) +
                 t13 * (t12 * t23 - t22 * t13);
    double* Ci = C + 6 * i;
    Ci[0] = (t22 * t33 - t23 * t23) / det;
    Ci[1] = (t13 * t23 - t12 * t33) / det;
    Ci[2] = (t12 * t23 - t13 * t22) / det;
    Ci[3] = (t11 * t33 - t13 * t13) / det;
    Ci[4] = (t12 * t13 - t11 * t23) / det;
    Ci[5] = (t11 * t22 - t12 * t12) / det;
    for (int e = 0; e < 6; ++e) { tau[6 * i + e] = t[e]; tau_abs[6 * i + e] = ta[e]; }
    if (!(det > 0.0) || !isfinite(det)) {
#pragma omp atomic write
      status = ORACLE_ERR_SINGULAR;
    }
  }
  return status;
}

/* C_i * v for the symmetric matrix stored as 11,12,13,22,23,33. */
static void sym_mul(const double* c, const double v[3], double out[3]) {
  out[0] = c[0] * v[0] + c[1] * v[1] + c[2] * v[2];
  out[1] = c[1] * v[0] + c[3] * v[1] + c[4] * v[2];
  out[2] = c[2] * v[0] + c[4] * v[1] + c[5] * v[2];
}

/* Monaghan artificial viscosity of one pair:
 *   mu = hbar rv / (d2 + eps hbar^2),
 *   Pi = (-alpha cbar mu + beta mu^2) / rhobar  if rv < 0, else 0. */
double oracle_av_pi(double rv, double d2, double hbar, double cbar, double rhobar,
                    const oracle_params* P) {
  if (!(rv < 0.0)) return 0.0;
  double mu = hbar * rv / (d2 + P->av_eps * hbar * hbar);
  return (-P->av_alpha * cbar * mu + P->av_beta * mu * mu) / rhobar;
}

/* ---------------------------------------------------------------------------
 * Step 8, momentum and energy (MomentumEnergy reading).  For j in N(i):
 *   w_i = W(r, h_i), w_j = W(r, h_j) (0 if r >= 2h_j)
 *   A = C_i Delta w_i,  B = C_j Delta w_j,  G = (A + B)/2
 *   v_ij = v_i - v_j;  rv = d . v_ij;  hbar, cbar, rhobar = arithmetic means
 *   a_i  = - sum_j m_j [ (p_i/rho_i^2) A + (p_j/rho_j^2) B + Pi G ]
 *   du_i =   sum_j m_j [ (p_i/rho_i^2) v_ij . A + (1/2) Pi v_ij . G ]
 * a_abs/du_abs: sum_j of the absolute values of every term (tolerance scale).
 * ------------------------------------------------------------------------- */
void oracle_momentum_energy(int64_t n, const double* x, const double* y, const double* z,
                            const double* vx, const double* vy, const double* vz,
                            const double* h, const double* m, const double* rho, const double* p,
                            const double* c, const double* C, const double bmin[3],
                            const double bmax[3], const int32_t per[3], const int64_t* off,
                            const int64_t* idx, const oracle_params* P, const double* fav,
                            const double* omega, double* ax, double* ay,
                            double* az, double* du, double* a_abs /* n x 3 */, double* du_abs) {
#pragma omp parallel for schedule(dynamic, 64)
  for (int64_t i = 0; i < n; ++i) {
    double acc[3] = {0, 0, 0}, accabs[3] = {0, 0, 0}, e = 0, eabs = 0;
    /* grad-h (reading 21): p/(Omega rho^2) in place of p/rho^2 */
    double pri = omega ? p[i] / (rho[i] * rho[i] * omega[i]) : p[i] / (rho[i] * rho[i]);
    for (int64_t k = off[i]; k < off[i + 1]; ++k) {
      int64_t j = idx[k];
      double d[3];
      double d2 = pair_d(x, y, z, i, j, bmin, bmax, per, d);
      double r = sqrt(d2);
      double D[3] = {-d[0], -d[1], -d[2]};
      double wi = oracle_W(r, h[i], P->K);
      double wj = oracle_W(r, h[j], P->K);
      double CiD[3], CjD[3];
      sym_mul(C + 6 * i, D, CiD);
      sym_mul(C + 6 * j, D, CjD);
      double A[3], B[3], G[3];
      for (int a = 0; a < 3; ++a) {
        A[a] = CiD[a] * wi;
        B[a] = CjD[a] * wj;
        G[a] = (A[a] + B[a]) / 2.0;
      }
      double vij[3] = {vx[i] - vx[j], vy[i] - vy[j], vz[i] - vz[j]};
      double rv = d[0] * vij[0] + d[1] * vij[1] + d[2] * vij[2];
      double hbar = (h[i] + h[j]) / 2.0;
      double cbar = (c[i] + c[j]) / 2.0;
      double rhobar = (rho[i] + rho[j]) / 2.0;
      double Pi = oracle_av_pi(rv, d2, hbar, cbar, rhobar, P);
      if (fav) Pi = Pi * ((fav[i] + fav[j]) / 2.0);  /* AV switch (reading 19) */
      double prj = omega ? p[j] / (rho[j] * rho[j] * omega[j]) : p[j] / (rho[j] * rho[j]);
      for (int a = 0; a < 3; ++a) {
        double t1 = pri * A[a], t2 = prj * B[a], t3 = Pi * G[a];
        acc[a] += -m[j] * (t1 + t2 + t3);
        accabs[a] += m[j] * (fabs(t1) + fabs(t2) + fabs(t3));
      }
      double vA = vij[0] * A[0] + vij[1] * A[1] + vij[2] * A[2];
      double vG = vij[0] * G[0] + vij[1] * G[1] + vij[2] * G[2];
      double e1 = pri * vA, e2 = 0.5 * Pi * vG;
      e += m[j] * (e1 + e2);
      eabs += m[j] * (fabs(e1) + fabs(e2));
    }
    ax[i] = acc[0];
    ay[i] = acc[1];
    az[i] = acc[2];
    du[i] = e;
    a_abs[3 * i + 0] = accabs[0];
    a_abs[3 * i + 1] = accabs[1];
    a_abs[3 * i + 2] = accabs[2];
    du_abs[i] = eabs;
  }
}

/* ---------------------------------------------------------------------------
 * Step 9, time step (the end-of-step collective of P:220):
 *   dt = min(C * min_i h_i / c_i,  growth * dt_prev).
 * ------------------------------------------------------------------------- */
double oracle_timestep(int64_t n, const double* h, const double* c, double dt_prev,
                       const oracle_params* P) {
  double m = INFINITY;
  for (int64_t i = 0; i < n; ++i) {
    double q = h[i] / c[i];
    if (q < m) m = q;
  }
  double a = P->k_cour * m, b = P->dt_max_growth * dt_prev;
  return a < b ? a : b;
}

/* ---------------------------------------------------------------------------
 * Step 9, signal-velocity variant (reading 22; optional):
 *   w_ij = min(0, v_ij . d_ij / r_ij)     (d = x_i - x_j, v_ij = v_i - v_j)
 *   vsig_i = max(2 c_i, max_{j in N(i)} (c_i + c_j - 3 w_ij))
 *   dt = min(C * min_i h_i / vsig_i,  growth * dt_prev).
 * vsig_out (may be NULL) receives vsig_i.
 * ------------------------------------------------------------------------- */
double oracle_timestep_vsig(int64_t n, const double* x, const double* y, const double* z,
                            const double* vx, const double* vy, const double* vz,
                            const double* h, const double* c, const double bmin[3],
                            const double bmax[3], const int32_t per[3], const int64_t* off,
                            const int64_t* idx, double dt_prev, const oracle_params* P,
                            double* vsig_out) {
  double m = INFINITY;
  for (int64_t i = 0; i < n; ++i) {
    double vs = 2.0 * c[i];
    for (int64_t k = off[i]; k < off[i + 1]; ++k) {
      int64_t j = idx[k];
      double d[3];
      double r = sqrt(pair_d(x, y, z, i, j, bmin, bmax, per, d));
      double rv = d[0] * (vx[i] - vx[j]) + d[1] * (vy[i] - vy[j]) + d[2] * (vz[i] - vz[j]);
      double w = rv < 0.0 ? rv / r : 0.0;
      double v = c[i] + c[j] - 3.0 * w;
      if (v > vs) vs = v;
    }
    if (vsig_out) vsig_out[i] = vs;
    double q = h[i] / vs;
    if (q < m) m = q;
  }
  double a = P->k_cour * m, b = P->dt_max_growth * dt_prev;
  return a < b ? a : b;
}

/* ---------------------------------------------------------------------------
 * Step 10, update (dt_m1 = dt of the previous step; first step: du_m1 := du).
 *   v <- v + a (dt + dt_m1)/2
 *   x <- x + v dt, then wrap periodic axes into [min, max) once
 *   u <- u + du (dt + dt^2/(2 dt_m1)) - du_m1 dt^2/(2 dt_m1);  du_m1 <- du
 *   h <- min(h * 1/2 * (1 + 1023 ng0 / max(nc,1))^(1/10), h_cap)
 * ------------------------------------------------------------------------- */
void oracle_update(int64_t n, double* x, double* y, double* z, double* vx, double* vy,
                   double* vz, double* h, double* u, double* du_m1, const double* ax,
                   const double* ay, const double* az, const double* du, const int32_t* nc,
                   double dt, double dt_m1, int first_step, const double bmin[3],
                   const double bmax[3], const oracle_params* P) {
  double* pos[3] = {x, y, z};
  double* vel[3] = {vx, vy, vz};
  const double* acc[3] = {ax, ay, az};
  for (int64_t i = 0; i < n; ++i) {
    for (int a = 0; a < 3; ++a) {
      vel[a][i] = vel[a][i] + acc[a][i] * (dt + dt_m1) / 2.0;
      pos[a][i] = pos[a][i] + vel[a][i] * dt;
      if (P->periodic[a]) {
        double L = bmax[a] - bmin[a];
        if (pos[a][i] >= bmax[a]) pos[a][i] -= L;
        else if (pos[a][i] < bmin[a]) pos[a][i] += L;
      }
    }
    double dum1 = first_step ? du[i] : du_m1[i];
    double half = dt * dt / (2.0 * dt_m1);
    u[i] = u[i] + du[i] * (dt + half) - dum1 * half;
    du_m1[i] = du[i];
    double ncd = nc[i] > 1 ? (double)nc[i] : 1.0;
    double hn = h[i] * 0.5 * pow(1.0 + 1023.0 * P->ng0 / ncd, 0.1);
    h[i] = hn < P->h_cap ? hn : P->h_cap;
  }
}

/* ---------------------------------------------------------------------------
 * Turbulence driving (Ornstein-Uhlenbeck stirring of the
 * Subsonic Turbulence workload).  PAPER.md prints no driving
 * formula; the definitions are the ones stated in include/sph.h and DESIGN.md
 * (reading 17), restated here:
 *   modes: integer n with 1 <= |n|^2 <= 9 in the half space (n_x > 0, or
 *          n_x = 0 and n_y > 0, or n_x = n_y = 0 and n_z > 0), lexicographic
 *          in (n_x, n_y, n_z); k_a = 2 pi n_a / L_a;
 *   OU:    A <- f A + sigma sqrt(1 - f^2) xi,  f = exp(-dt / t_decay);
 *   projection: A^ = zeta (A - k^(k^.A)) + (1 - zeta) k^(k^.A), applied to the
 *          real and the imaginary 3-vector of each mode; B = 2 w A^;
 *   acceleration: a_i += sum_m [ Re(B_m) cos(phi) - Im(B_m) sin(phi) ],
 *          phi = k_m . (x_i - box_min).
 * A mode's 6 numbers are (Re x, Im x, Re y, Im y, Re z, Im z).
 * ------------------------------------------------------------------------- */
int oracle_stir_modes(int32_t* n3) {
  int m = 0;
  for (int nx = 0; nx <= 3; ++nx)
    for (int ny = -3; ny <= 3; ++ny)
      for (int nz = -3; nz <= 3; ++nz) {
        int q = nx * nx + ny * ny + nz * nz;
        int half = nx > 0 || (nx == 0 && ny > 0) || (nx == 0 && ny == 0 && nz > 0);
        if (half && q >= 1 && q <= 9) {
          n3[3 * m + 0] = nx;
          n3[3 * m + 1] = ny;
          n3[3 * m + 2] = nz;
          ++m;
        }
      }
  return m;
}

void oracle_stir_ou(int nm, double* A, const double* xi, double dt, double sigma, double t_decay) {
  double f = exp(-dt / t_decay);
  double g = sigma * sqrt(1.0 - f * f);
  for (int k = 0; k < 6 * nm; ++k) A[k] = f * A[k] + g * xi[k];
}

void oracle_stir_project(int nm, const int32_t* n3, const double L[3], const double* A,
                         const double* w, double zeta, double* B) {
  for (int m = 0; m < nm; ++m) {
    double k[3], kn = 0.0;
    for (int a = 0; a < 3; ++a) {
      k[a] = 2.0 * M_PI * n3[3 * m + a] / L[a];
      kn += k[a] * k[a];
    }
    kn = sqrt(kn);
    for (int a = 0; a < 3; ++a) k[a] /= kn;
    for (int part = 0; part < 2; ++part) {
      double v[3], kv = 0.0;
      for (int a = 0; a < 3; ++a) {
        v[a] = A[6 * m + 2 * a + part];
        kv += k[a] * v[a];
      }
      for (int a = 0; a < 3; ++a) {
        double par = k[a] * kv;
        double perp = v[a] - par;
        B[6 * m + 2 * a + part] = 2.0 * w[m] * (zeta * perp + (1.0 - zeta) * par);
      }
    }
  }
}

void oracle_stir_accel(int64_t n, const double* x, const double* y, const double* z,
                       const double lo[3], const double L[3], int nm, const int32_t* n3,
                       const double* B, double* ax, double* ay, double* az) {
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < n; ++i) {
    double s[3] = {0.0, 0.0, 0.0};
    const double p[3] = {x[i] - lo[0], y[i] - lo[1], z[i] - lo[2]};
    for (int m = 0; m < nm; ++m) {
      double phi = 0.0;
      for (int a = 0; a < 3; ++a) phi += 2.0 * M_PI * n3[3 * m + a] * p[a] / L[a];
      double c = cos(phi), sn = sin(phi);
      for (int a = 0; a < 3; ++a) s[a] += B[6 * m + 2 * a] * c - B[6 * m + 2 * a + 1] * sn;
    }
    ax[i] += s[0];
    ay[i] += s[1];
    az[i] += s[2];
  }
}

/* ---------------------------------------------------------------------------
 * Velocity divergence and curl of IADVelocityDivCurl (SURVEY 8(f)-1,
 * DESIGN.md reading 19).  The IAD gradient of a field f at particle i is
 *   (grad f)_i = sum_j V_j W(r_ij, h_i) (C_i Delta_ij) (f_j - f_i),
 *   V_j = m_j / rho_j, Delta_ij = x_j - x_i (minimum image),
 * exact for linear f (C_i = tau_i^-1).  Applied to the velocity it gives the
 * tensor T_ab = d v_b / d x_a:
 *   T_ab = sum_j V_j W(r_ij, h_i) (C_i Delta_ij)_a (v_j - v_i)_b,
 *   div v = T_xx + T_yy + T_zz,
 *   curl v = (T_yz - T_zy, T_zx - T_xz, T_xy - T_yx).
 * T_abs holds sum_j |term_ab| (the tolerance scale).
 * ------------------------------------------------------------------------- */
void oracle_divcurl(int64_t n, const double* x, const double* y, const double* z,
                    const double* vx, const double* vy, const double* vz, const double* h,
                    const double* m, const double* rho, const double* C, const double bmin[3],
                    const double bmax[3], const int32_t per[3], const int64_t* off,
                    const int64_t* idx, const oracle_params* P, double* T /* n x 9 */,
                    double* T_abs /* n x 9 */, double* divv, double* curl /* n x 3 */) {
#pragma omp parallel for schedule(dynamic, 64)
  for (int64_t i = 0; i < n; ++i) {
    double t[9] = {0, 0, 0, 0, 0, 0, 0, 0, 0}, ta[9] = {0, 0, 0, 0, 0, 0, 0, 0, 0};
    for (int64_t k = off[i]; k < off[i + 1]; ++k) {
      int64_t j = idx[k];
      double d[3];
      double r = sqrt(pair_d(x, y, z, i, j, bmin, bmax, per, d));
      double D[3] = {-d[0], -d[1], -d[2]};
      double CD[3];
      sym_mul(C + 6 * i, D, CD);
      double vw = (m[j] / rho[j]) * oracle_W(r, h[i], P->K);
      double dv[3] = {vx[j] - vx[i], vy[j] - vy[i], vz[j] - vz[i]};
      for (int a = 0; a < 3; ++a)
        for (int b = 0; b < 3; ++b) {
          double term = vw * CD[a] * dv[b];
          t[3 * a + b] += term;
          ta[3 * a + b] += fabs(term);
        }
    }
    for (int e = 0; e < 9; ++e) { T[9 * i + e] = t[e]; T_abs[9 * i + e] = ta[e]; }
    divv[i] = t[0] + t[4] + t[8];
    curl[3 * i + 0] = t[5] - t[7];  /* dv_z/dy - dv_y/dz */
    curl[3 * i + 1] = t[6] - t[2];  /* dv_x/dz - dv_z/dx */
    curl[3 * i + 2] = t[1] - t[3];  /* dv_y/dx - dv_x/dy */
  }
}

/* Balsara (1995) switch: f_i = |div v| / (|div v| + |curl v| + 1e-4 c_i / h_i);
 * the artificial viscosity of a pair is multiplied by (f_i + f_j) / 2. */
void oracle_balsara(int64_t n, const double* divv, const double* curl, const double* c,
                    const double* h, double* f) {
  for (int64_t i = 0; i < n; ++i) {
    double ad = fabs(divv[i]);
    double ac = sqrt(curl[3 * i] * curl[3 * i] + curl[3 * i + 1] * curl[3 * i + 1] +
                     curl[3 * i + 2] * curl[3 * i + 2]);
    f[i] = ad / (ad + ac + 1e-4 * c[i] / h[i]);
  }
}

/* ---------------------------------------------------------------------------
 * Self-gravity (the Evrard collapse workload, P:108, P:135;
 * DESIGN.md reading 20).  Newtonian attraction with Plummer softening eps,
 * isolated (open) boundaries, by direct summation over j != i in ascending
 * order -- the definition the GPU tree code approximates:
 *   a_i   = G sum_j m_j (x_j - x_i) / (|x_j - x_i|^2 + eps^2)^(3/2),
 *   phi_i = -G sum_j m_j / (|x_j - x_i|^2 + eps^2)^(1/2).
 * a_abs[3i+a] = sum_j |term_a| (the tolerance scale).
 * ------------------------------------------------------------------------- */
void oracle_gravity(int64_t n, const double* x, const double* y, const double* z,
                    const double* m, double G, double eps, double* ax, double* ay, double* az,
                    double* phi, double* a_abs) {
#pragma omp parallel for schedule(dynamic, 16)
  for (int64_t i = 0; i < n; ++i) {
    double a[3] = {0, 0, 0}, aa[3] = {0, 0, 0}, p = 0.0;
    for (int64_t j = 0; j < n; ++j) {
      if (j == i) continue;
      double d[3] = {x[j] - x[i], y[j] - y[i], z[j] - z[i]};
      double r2 = d[0] * d[0] + d[1] * d[1] + d[2] * d[2] + eps * eps;
      double r = sqrt(r2);
      double s = G * m[j] / (r2 * r);
      for (int c = 0; c < 3; ++c) {
        a[c] += s * d[c];
        aa[c] += fabs(s * d[c]);
      }
      p -= G * m[j] / r;
    }
    ax[i] = a[0];
    ay[i] = a[1];
    az[i] = a[2];
    phi[i] = p;
    for (int c = 0; c < 3; ++c) a_abs[3 * i + c] = aa[c];
  }
}
