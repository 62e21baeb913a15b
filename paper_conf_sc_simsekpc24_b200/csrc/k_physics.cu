// k_physics.cu -- phases DENSITY, EOS, IAD, MOMENTUM_ENERGY, TIMESTEP, UPDATE
// (items 5-10 of DESIGN.md section 3; the paper's XMass P:184,
// IADVelocityDivCurl P:180, MomentumEnergy P:160/P:180, the end-of-step
// collective P:220).
//
// The three neighbour sums run one thread per target over its stored list in
// list order (ascending j, the oracle's summation order).  Lists are column-
// major so the k-th neighbour indices of a warp's 32 consecutive targets are one
// coalesced 128-B load.  The j-side data are gathered as packed 32-byte records
// (one 256-bit load each; see Rec4 in sph_internal.cuh), built by the phase that
// produces their last field: rec_d by the sort's permutation, rec_i by EOS,
// rec_m by IAD.  Consecutive targets share most neighbours (Morton order), so the
// gathers hit L1/L2.  The sinc kernel is a polynomial in t = r^2 (pi/2h)^2 (no
// sqrt/sin per pair); (pi/2h)^2 and K/h^3 are computed once per particle by the
// density kernel.  All three sums are FP64-bound.
#include <algorithm>

#include "sph_internal.cuh"

namespace sph {

// diagnostic builds only (SPH_NVCC_EXTRA=-DSPH_MOM_DIAG=1 / 2): the
// momentum-energy loop with its gathers alone / its arithmetic alone
#ifndef SPH_MOM_DIAG
#define SPH_MOM_DIAG 0
#endif


// Neighbour-list index loads (A/B builds, SPH_IDX_POLICY): 0 = ld.global.nc;
// 1 = L1::no_allocate (each list line is used once, by the whole warp at once:
// keep L1 for the gathered records); 2 = L1::evict_first.
#ifndef SPH_IDX_POLICY
#define SPH_IDX_POLICY 1
#endif
__device__ __forceinline__ int ldg_idx(const int32_t* p) {
#if SPH_IDX_POLICY == 1
  int v;
  asm("ld.global.nc.L1::no_allocate.b32 %0, [%1];" : "=r"(v) : "l"(p));
  return v;
#elif SPH_IDX_POLICY == 2
  int v;
  asm("ld.global.nc.L1::evict_first.b32 %0, [%1];" : "=r"(v) : "l"(p));
  return v;
#else
  return __ldg(p);
#endif
}

constexpr double kPi = 3.14159265358979323846;
constexpr double kPi2Over4 = kPi * kPi / 4.0;
constexpr double kPi2 = kPi * kPi;

// Block sizes of the neighbour sums: one large CTA per SM (the register file
// allows 1024 x 64, 768 x 85, 512 x 128) keeps an SM on one run of consecutive
// (Morton-adjacent) targets, so the gathered records of its warps overlap in L1
// instead of coming from several distant regions (momentum 11.5 -> 11.0 ms; a
// persistent contiguous-range grid was slower: spills and tail imbalance).
#ifndef SPH_DENS_THREADS
#define SPH_DENS_THREADS 1024  // A/B builds only
#endif
constexpr int kDensThreads = SPH_DENS_THREADS;
#ifndef SPH_IAD_THREADS
#define SPH_IAD_THREADS 768  // A/B builds only
#endif
constexpr int kIadThreads = SPH_IAD_THREADS;
// A/B builds only: other CTA sizes of momentum-energy
#ifndef SPH_MOM_THREADS
#define SPH_MOM_THREADS 512
#endif
constexpr int kMomThreads = SPH_MOM_THREADS;

struct Geom {
  double L[3], H[3], lo[3], hi[3];
  bool per[3];
};

__device__ __forceinline__ Geom load_geom(const DevScalars* ds, const Params& P) {
  Geom g;
#pragma unroll
  for (int a = 0; a < 3; ++a) {
    g.L[a] = ds->box_max[a] - ds->box_min[a];
    g.H[a] = 0.5 * g.L[a];
    g.per[a] = P.periodic[a] != 0;
    g.lo[a] = ds->box_min[a];
    g.hi[a] = ds->box_max[a];
  }
  return g;
}

// True unless every neighbour of a target at x with smoothing length h is
// certainly reached without a periodic image: a neighbour needs the image only
// if |x_i - x_j| > L - 2h_i, impossible when x_i is >= 2h_i from both faces
// (2.5 h keeps a margin for rounding).  Then the oracle's conditional +-L never
// fires and d = x_i - x_j is the same double.
__device__ __forceinline__ bool needs_wrap(const Geom& g, double x, double y, double z, double h) {
  const double m = 2.5 * h;
  const double c[3] = {x, y, z};
  bool w = false;
#pragma unroll
  for (int a = 0; a < 3; ++a)
    if (g.per[a] && (c[a] - g.lo[a] < m || g.hi[a] - c[a] < m)) w = true;
  return w;
}

// d = x_i - x_j, minimum image (the oracle's order: raw difference, then +-L);
// kWrap = false for warps whose targets all pass needs_wrap() == false.
template <bool kWrap>
__device__ __forceinline__ void pair_d(const Geom& g, double xi, double yi, double zi, double xj,
                                       double yj, double zj, double& dx, double& dy, double& dz) {
  if (kWrap) {
    dx = min_image(xi - xj, g.L[0], g.H[0], g.per[0]);
    dy = min_image(yi - yj, g.L[1], g.H[1], g.per[1]);
    dz = min_image(zi - zj, g.L[2], g.H[2], g.per[2]);
  } else {
    dx = xi - xj;
    dy = yi - yj;
    dz = zi - zj;
  }
}

// ------------------------------------------------------------------ density
// rho_i = (K/h_i^3) [m_i + sum_j m_j S(pi r_ij / 2h_i)^6]; also writes the
// per-particle kernel factors wq = (pi/2h)^2 and wk = K/h^3 reused by IAD and
// momentum-energy.  Per pair: one 32-B record {x, y, z, m}, 40 DP flops.
template <bool kWrap>
__device__ __forceinline__ void density_body(const Fields& F, const Params& P, const Geom& g, int64_t i,
                                             const Rec4& me, double hi) {
  const double q = kPi2Over4 / (hi * hi);
  const double kh3 = P.K / (hi * hi * hi);
  const int nci = min(F.nc[i], F.ngmax);
  double sum = me.d;
  const int32_t* __restrict__ nb = F.nbr + i;
  const Rec4* __restrict__ rec = F.rec_d;
  // two neighbours per iteration (two independent sinc chains in flight; the sum
  // is still accumulated in list order), records one pair ahead, indices two
  const int64_t cap = F.cap;
  Rec4 ra = ldg4(rec + (nci > 0 ? ldg_idx(nb) : 0)), rb = ldg4(rec + (nci > 1 ? ldg_idx(nb + cap) : 0));
  int jc = nci > 2 ? ldg_idx(nb + 2 * cap) : 0, jd = nci > 3 ? ldg_idx(nb + 3 * cap) : 0;
  int k = 0;
  for (; k + 1 < nci; k += 2) {
    const Rec4 a = ra, b = rb;
    if (k + 2 < nci) ra = ldg4(rec + jc);
    if (k + 3 < nci) rb = ldg4(rec + jd);
    if (k + 4 < nci) jc = ldg_idx(nb + (int64_t)(k + 4) * cap);
    if (k + 5 < nci) jd = ldg_idx(nb + (int64_t)(k + 5) * cap);
    double dxa, dya, dza, dxb, dyb, dzb;
    pair_d<kWrap>(g, me.a, me.b, me.c, a.a, a.b, a.c, dxa, dya, dza);
    pair_d<kWrap>(g, me.a, me.b, me.c, b.a, b.b, b.c, dxb, dyb, dzb);
    const double sa = sinc6_t((dxa * dxa + dya * dya + dza * dza) * q);
    const double sb = sinc6_t((dxb * dxb + dyb * dyb + dzb * dzb) * q);
    sum = fma(a.d, sa, sum);
    sum = fma(b.d, sb, sum);
  }
  if (k < nci) {
    double dx, dy, dz;
    pair_d<kWrap>(g, me.a, me.b, me.c, ra.a, ra.b, ra.c, dx, dy, dz);
    sum = fma(ra.d, sinc6_t((dx * dx + dy * dy + dz * dz) * q), sum);
  }
  F.rho[i] = kh3 * sum;
  F.wq[i] = q;
  F.wk[i] = kh3;
}

// Ghosts (another rank's particles, SPH_GHOST_BIT in the id) are neighbours j
// only: their own sums would use a truncated neighbourhood and are replaced by
// the owners' values (halo), so the neighbour sums skip them as targets and
// write only what the j side reads (kernel factors here, the momentum record in
// IAD).
__device__ __forceinline__ bool is_ghost(const Fields& F, int64_t i) { return (F.id[i] & SPH_GHOST_BIT) != 0; }

// Target classes of a split IAD / MOMENTUM_ENERGY (sph_set_part, multi-rank
// overlap): INTERIOR = no ghost among the neighbours (can run before the halo
// values arrive), BOUNDARY = the rest (+ the ghosts' momentum records in IAD).
__device__ __forceinline__ bool in_part(const Fields& F, int part, int64_t i) {
  return part == SPH_PART_ALL || (part == SPH_PART_INTERIOR ? F.bnd[i] == 0 : F.bnd[i] != 0);
}

// The momentum record of a ghost (its C comes from the owner: halo, then
// refresh_rec_m rewrites the C chunks).
__device__ __forceinline__ void ghost_rec_m(const Fields& F, int64_t i, const Rec4& me) {
  Rec4* rm = F.rec_m + (int64_t)kRecM * i;
  st4(rm + 0, me.a, me.b, me.c, F.wq[i]);
  st4(rm + 1, 0.0, 0.0, 0.0, F.wk[i]);
  st4(rm + 2, 0.0, 0.0, 0.0, F.f[FM][i]);
  st4(rm + 3, F.f[FVX][i], F.f[FVY][i], F.f[FVZ][i], F.prho2[i]);
  st4(rm + 4, F.f[FH][i], F.c[i], F.rho[i], 1.0);
}


__global__ void __launch_bounds__(kDensThreads, 1024 / kDensThreads) density_kernel(Fields F, Params P) {
  const int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (i >= F.n) return;
  const Geom g = load_geom(F.ds, P);
  const Rec4 me = F.rec_d[i];
  const double hi = F.f[FH][i];
  if (is_ghost(F, i)) {
    F.wq[i] = kPi2Over4 / (hi * hi);
    F.wk[i] = P.K / (hi * hi * hi);
    return;
  }
  if (__any_sync(__activemask(), needs_wrap(g, me.a, me.b, me.c, hi)))
    density_body<true>(F, P, g, i, me, hi);
  else
    density_body<false>(F, P, g, i, me, hi);
}

// ------------------------------------------------------------------ EOS
// Bit-exact vs the oracle (same operation order, IEEE sqrt/div): p, c; plus the
// derived V = m/rho, p/rho^2 and the IAD record {x, y, z, V}.
__global__ void __launch_bounds__(256) eos_kernel(Fields F, Params P, bool apply_omega) {
  const int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (i >= F.n) return;
  if (P.part == SPH_PART_GHOSTS && !is_ghost(F, i)) return;  // the ghosts' EOS after the rho halo
  const double rho = F.rho[i], u = F.f[FU][i];
  double p, c;
  if (P.eos == SPH_EOS_IDEAL) {
    p = __dmul_rn(__dmul_rn(P.gamma - 1.0, rho), u);
    c = __dsqrt_rn(__dmul_rn(__dmul_rn(P.gamma, P.gamma - 1.0), u));
  } else {
    p = __dmul_rn(__dmul_rn(P.cs0, P.cs0), rho);
    c = P.cs0;
  }
  const Rec4 rd = F.rec_d[i];
  const double V = __ddiv_rn(rd.d, rho);
  F.p[i] = p;
  F.c[i] = c;
  F.vol[i] = V;
  // after a volume-element GRADH (reading 23) the grad-h factor is already known
  F.prho2[i] = apply_omega ? __ddiv_rn(p, __dmul_rn(__dmul_rn(rho, rho), F.omega[i]))
                           : __ddiv_rn(p, __dmul_rn(rho, rho));
  st4(F.rec_i + i, rd.a, rd.b, rd.c, V);
  if (P.divcurl) st4(F.rec_iv + i, F.f[FVX][i], F.f[FVY][i], F.f[FVZ][i], 0.0);
}

// ------------------------------------------------------------------ GRADH
// NormalizationGradh (reading 21): Omega_i = 1 + (h_i/(3 rho_i)) sum_j m_j dW/dh,
// dW/dh = -(K/h^4) S^5 (6 cos x - 3 S), x = pi r/2h, self term 3 m_i inside the
// bracket.  S and cos x are polynomials in t = x^2 = r^2 (pi/2h)^2 (no sqrt,
// sin or cos per pair); then p/rho^2 -> p/(Omega rho^2) for the momentum
// records (written by IAD).  Per pair: one 32-B record {x, y, z, m} (the
// density record), two neighbours per iteration like DENSITY.
__device__ __forceinline__ double dwdh_term(double t) {
  const double S = sinc_t(t), S2 = S * S;
  return (S2 * S2 * S) * fma(6.0, cos_t(t), -3.0 * S);
}

template <bool kWrap, bool kVE>
__device__ __forceinline__ void gradh_body(const Fields& F, const Params& P, const Geom& g, int64_t i,
                                           const Rec4& me, double hi) {
  // records {x, y, z, w}: w = m (plain) or X = V0 = m/rho0 (volume elements,
  // the EOS's IAD record, reading 23)
  const int nci = min(F.nc[i], F.ngmax);
  const double q = F.wq[i];
  double sum = 3.0 * me.d;  // dW/dh bracket, self: S = 1, cos = 1
  double sw = me.d;         // normalisation sum (kVE), self: S^6 = 1
  const int32_t* __restrict__ nb = F.nbr + i;
  const Rec4* __restrict__ rec = kVE ? F.rec_i : F.rec_d;
  const int64_t cap = F.cap;
  auto add = [&](const Rec4& rj, double t) {
    const double S = sinc_t(t), S2 = S * S, S5 = S2 * S2 * S;
    sum = fma(rj.d * S5, fma(6.0, cos_t(t), -3.0 * S), sum);
    if (kVE) sw = fma(rj.d, S5 * S, sw);
  };
  Rec4 ra = ldg4(rec + (nci > 0 ? ldg_idx(nb) : 0)), rb = ldg4(rec + (nci > 1 ? ldg_idx(nb + cap) : 0));
  int jc = nci > 2 ? ldg_idx(nb + 2 * cap) : 0, jd = nci > 3 ? ldg_idx(nb + 3 * cap) : 0;
  int k = 0;
  for (; k + 1 < nci; k += 2) {
    const Rec4 a = ra, b = rb;
    if (k + 2 < nci) ra = ldg4(rec + jc);
    if (k + 3 < nci) rb = ldg4(rec + jd);
    if (k + 4 < nci) jc = ldg_idx(nb + (int64_t)(k + 4) * cap);
    if (k + 5 < nci) jd = ldg_idx(nb + (int64_t)(k + 5) * cap);
    double dxa, dya, dza, dxb, dyb, dzb;
    pair_d<kWrap>(g, me.a, me.b, me.c, a.a, a.b, a.c, dxa, dya, dza);
    pair_d<kWrap>(g, me.a, me.b, me.c, b.a, b.b, b.c, dxb, dyb, dzb);
    add(a, (dxa * dxa + dya * dya + dza * dza) * q);
    add(b, (dxb * dxb + dyb * dyb + dzb * dzb) * q);
  }
  if (k < nci) {
    double dx, dy, dz;
    pair_d<kWrap>(g, me.a, me.b, me.c, ra.a, ra.b, ra.c, dx, dy, dz);
    add(ra, (dx * dx + dy * dy + dz * dz) * q);
  }
  double rho = F.rho[i];
  const double h2 = hi * hi;
  if (kVE) {
    const double kx = P.K / (h2 * hi) * sw;
    F.rho[i] = kx * F.f[FM][i] / me.d;  // rho = kx m / X
    rho = kx;                            // Omega uses kx in place of rho
  }
  if (P.gradh) {
    const double dsum = -P.K / (h2 * h2) * sum;
    const double om = 1.0 + hi / (3.0 * rho) * dsum;
    F.omega[i] = om;
    if (!kVE) F.prho2[i] = __ddiv_rn(F.p[i], __dmul_rn(__dmul_rn(rho, rho), om));
  }
}

__global__ void __launch_bounds__(kDensThreads, 1024 / kDensThreads) gradh_kernel(Fields F, Params P) {
  const int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (i >= F.n) return;
  const Geom g = load_geom(F.ds, P);
  const double hi = F.f[FH][i];
  if (is_ghost(F, i)) return;  // rho and Omega of a ghost come from its owner (halo)
  if (P.ve) {
    const Rec4 me = F.rec_i[i];
    if (__any_sync(__activemask(), needs_wrap(g, me.a, me.b, me.c, hi)))
      gradh_body<true, true>(F, P, g, i, me, hi);
    else
      gradh_body<false, true>(F, P, g, i, me, hi);
  } else {
    const Rec4 me = F.rec_d[i];
    if (__any_sync(__activemask(), needs_wrap(g, me.a, me.b, me.c, hi)))
      gradh_body<true, false>(F, P, g, i, me, hi);
    else
      gradh_body<false, false>(F, P, g, i, me, hi);
  }
}

// p/(Omega rho^2) again after sph_set_field wrote the owners' Omega over the
// ghosts (multi-GPU halo).
__global__ void __launch_bounds__(256) prho2_kernel(Fields F) {
  const int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (i >= F.n) return;
  const double rho = F.rho[i];
  F.prho2[i] = __ddiv_rn(F.p[i], __dmul_rn(__dmul_rn(rho, rho), F.omega[i]));
}

// ------------------------------------------------------------------ IAD
// tau_i = sum_j V_j W(r,h_i) Delta Delta^T, C_i = tau_i^{-1} (adjugate / det);
// epilogue: the momentum record of particle i.  Per pair: one 32-B record
// {x, y, z, V}, 55 DP flops.
template <bool kWrap>
__device__ __forceinline__ void iad_body(const Fields& F, const Geom& g, int64_t i, const Rec4& me) {
  const double q = F.wq[i], kh3 = F.wk[i];
  const int nci = min(F.nc[i], F.ngmax);
  double t11 = 0, t12 = 0, t13 = 0, t22 = 0, t23 = 0, t33 = 0;
  const int32_t* __restrict__ nb = F.nbr + i;
  const Rec4* __restrict__ rec = F.rec_i;
  // two neighbours per iteration (independent sinc chains in flight; the sums
  // are still accumulated in list order), records one pair ahead, indices two
  const int64_t cap = F.cap;
  auto add = [&](const Rec4& rj) {
    double dx, dy, dz;
    pair_d<kWrap>(g, me.a, me.b, me.c, rj.a, rj.b, rj.c, dx, dy, dz);
    const double r2 = dx * dx + dy * dy + dz * dz;
    const double vw = rj.d * (kh3 * sinc6_t(r2 * q));
    // Delta = -d; the products Delta^a Delta^b equal d^a d^b.
    const double ax = vw * dx, ay = vw * dy, az = vw * dz;
    t11 = fma(ax, dx, t11);
    t12 = fma(ax, dy, t12);
    t13 = fma(ax, dz, t13);
    t22 = fma(ay, dy, t22);
    t23 = fma(ay, dz, t23);
    t33 = fma(az, dz, t33);
  };
  Rec4 ra = ldg4(rec + (nci > 0 ? ldg_idx(nb) : 0)), rb = ldg4(rec + (nci > 1 ? ldg_idx(nb + cap) : 0));
  int jc = nci > 2 ? ldg_idx(nb + 2 * cap) : 0, jd = nci > 3 ? ldg_idx(nb + 3 * cap) : 0;
  int k = 0;
  for (; k + 1 < nci; k += 2) {
    const Rec4 a = ra, b = rb;
    if (k + 2 < nci) ra = ldg4(rec + jc);
    if (k + 3 < nci) rb = ldg4(rec + jd);
    if (k + 4 < nci) jc = ldg_idx(nb + (int64_t)(k + 4) * cap);
    if (k + 5 < nci) jd = ldg_idx(nb + (int64_t)(k + 5) * cap);
    add(a);
    add(b);
  }
  if (k < nci) add(ra);
  const double det = t11 * (t22 * t33 - t23 * t23) - t12 * (t12 * t33 - t23 * t13) +
                     t13 * (t12 * t23 - t22 * t13);
  const double inv = 1.0 / det;
  const double c11 = (t22 * t33 - t23 * t23) * inv, c12 = (t13 * t23 - t12 * t33) * inv;
  const double c13 = (t12 * t23 - t13 * t22) * inv, c22 = (t11 * t33 - t13 * t13) * inv;
  const double c23 = (t12 * t13 - t11 * t23) * inv, c33 = (t11 * t22 - t12 * t12) * inv;
  F.C[0][i] = c11;
  F.C[1][i] = c12;
  F.C[2][i] = c13;
  F.C[3][i] = c22;
  F.C[4][i] = c23;
  F.C[5][i] = c33;
  // ghosts (another rank's particles, SPH_GHOST_BIT in the id) have truncated
  // neighbourhoods; their C is overwritten by the owner's
  if ((!(det > 0.0) || !isfinite(det)) && !(F.id[i] & SPH_GHOST_BIT))
    atomicOr(&F.ds->status, (int)ST_SINGULAR);
  Rec4* rm = F.rec_m + (int64_t)kRecM * i;
  st4(rm + 0, me.a, me.b, me.c, q);
  st4(rm + 1, c11, c12, c13, kh3);
  st4(rm + 2, c22, c23, c33, F.f[FM][i]);
  st4(rm + 3, F.f[FVX][i], F.f[FVY][i], F.f[FVZ][i], F.prho2[i]);
  st4(rm + 4, F.f[FH][i], F.c[i], F.rho[i], 1.0);  // AV switch factor 1 (no switch)
}

// IADVelocityDivCurl with the velocity part (cfg.divcurl, reading 19): the same
// list walk also accumulates M = sum_j V_j W Delta (v_j - v_i)^T (9 sums; one
// more 32-B record {vx, vy, vz, 0} per pair), then T = C M (T_ab = dv_b/dx_a),
// div v = tr T, curl v from the antisymmetric part, and the Balsara factor.
template <bool kWrap>
__device__ __forceinline__ void iad_dc_body(const Fields& F, const Params& P, const Geom& g, int64_t i,
                                            const Rec4& me) {
  const double q = F.wq[i], kh3 = F.wk[i];
  const int nci = min(F.nc[i], F.ngmax);
  const double vxi = F.f[FVX][i], vyi = F.f[FVY][i], vzi = F.f[FVZ][i];
  double t11 = 0, t12 = 0, t13 = 0, t22 = 0, t23 = 0, t33 = 0;
  double M[3][3] = {{0, 0, 0}, {0, 0, 0}, {0, 0, 0}};
  const int32_t* __restrict__ nb = F.nbr + i;
  const Rec4* __restrict__ rec = F.rec_i;
  const Rec4* __restrict__ rv = F.rec_iv;
  const int64_t cap = F.cap;
  auto add = [&](const Rec4& rj, const Rec4& vj) {
    double dx, dy, dz;
    pair_d<kWrap>(g, me.a, me.b, me.c, rj.a, rj.b, rj.c, dx, dy, dz);
    const double r2 = dx * dx + dy * dy + dz * dz;
    const double vw = rj.d * (kh3 * sinc6_t(r2 * q));
    const double ax = vw * dx, ay = vw * dy, az = vw * dz;
    t11 = fma(ax, dx, t11);
    t12 = fma(ax, dy, t12);
    t13 = fma(ax, dz, t13);
    t22 = fma(ay, dy, t22);
    t23 = fma(ay, dz, t23);
    t33 = fma(az, dz, t33);
    // M_ab += V W Delta_a dv_b with Delta = -d
    const double dv[3] = {vj.a - vxi, vj.b - vyi, vj.c - vzi};
    const double aw[3] = {ax, ay, az};
#pragma unroll
    for (int a = 0; a < 3; ++a)
#pragma unroll
      for (int b = 0; b < 3; ++b) M[a][b] = fma(-aw[a], dv[b], M[a][b]);
  };
  // two neighbours per iteration (as iad_body), records one pair ahead,
  // indices two ahead; the sums still run in list order
  int j0 = nci > 0 ? ldg_idx(nb) : 0, j1 = nci > 1 ? ldg_idx(nb + cap) : 0;
  Rec4 ra = ldg4(rec + j0), va = ldg4(rv + j0), rb = ldg4(rec + j1), vb = ldg4(rv + j1);
  int jc = nci > 2 ? ldg_idx(nb + 2 * cap) : 0, jd = nci > 3 ? ldg_idx(nb + 3 * cap) : 0;
  int k = 0;
  for (; k + 1 < nci; k += 2) {
    const Rec4 a = ra, av = va, b = rb, bv = vb;
    if (k + 2 < nci) {
      ra = ldg4(rec + jc);
      va = ldg4(rv + jc);
    }
    if (k + 3 < nci) {
      rb = ldg4(rec + jd);
      vb = ldg4(rv + jd);
    }
    if (k + 4 < nci) jc = ldg_idx(nb + (int64_t)(k + 4) * cap);
    if (k + 5 < nci) jd = ldg_idx(nb + (int64_t)(k + 5) * cap);
    add(a, av);
    add(b, bv);
  }
  if (k < nci) add(ra, va);
  const double det = t11 * (t22 * t33 - t23 * t23) - t12 * (t12 * t33 - t23 * t13) +
                     t13 * (t12 * t23 - t22 * t13);
  const double inv = 1.0 / det;
  const double c11 = (t22 * t33 - t23 * t23) * inv, c12 = (t13 * t23 - t12 * t33) * inv;
  const double c13 = (t12 * t23 - t13 * t22) * inv, c22 = (t11 * t33 - t13 * t13) * inv;
  const double c23 = (t12 * t13 - t11 * t23) * inv, c33 = (t11 * t22 - t12 * t12) * inv;
  F.C[0][i] = c11;
  F.C[1][i] = c12;
  F.C[2][i] = c13;
  F.C[3][i] = c22;
  F.C[4][i] = c23;
  F.C[5][i] = c33;
  if ((!(det > 0.0) || !isfinite(det)) && !(F.id[i] & SPH_GHOST_BIT))
    atomicOr(&F.ds->status, (int)ST_SINGULAR);
  const double Cm[3][3] = {{c11, c12, c13}, {c12, c22, c23}, {c13, c23, c33}};
  double T[3][3];
#pragma unroll
  for (int a = 0; a < 3; ++a)
#pragma unroll
    for (int b = 0; b < 3; ++b) T[a][b] = Cm[a][0] * M[0][b] + Cm[a][1] * M[1][b] + Cm[a][2] * M[2][b];
  const double div = T[0][0] + T[1][1] + T[2][2];
  const double cx = T[1][2] - T[2][1], cy = T[2][0] - T[0][2], cz = T[0][1] - T[1][0];
  F.divv[i] = div;
  F.curl[0][i] = cx;
  F.curl[1][i] = cy;
  F.curl[2][i] = cz;
  double f = 1.0;
  if (P.av_switch) {
    const double ad = fabs(div), ac = sqrt(cx * cx + cy * cy + cz * cz);
    f = ad / (ad + ac + 1e-4 * F.c[i] / F.f[FH][i]);
    F.bal[i] = f;
  }
  Rec4* rm = F.rec_m + (int64_t)kRecM * i;
  st4(rm + 0, me.a, me.b, me.c, q);
  st4(rm + 1, c11, c12, c13, kh3);
  st4(rm + 2, c22, c23, c33, F.f[FM][i]);
  st4(rm + 3, vxi, vyi, vzi, F.prho2[i]);
  st4(rm + 4, F.f[FH][i], F.c[i], F.rho[i], f);
}

// 512 threads x 128 registers (640 x 102 spills with the two-pair loop;
// one pair per iteration: 512 -> 6.02, 640 -> 5.53 ms; two pairs at 512: 4.78)
#ifndef SPH_IADDC_THREADS
#define SPH_IADDC_THREADS 512  // A/B builds only
#endif
constexpr int kIadDcThreads = SPH_IADDC_THREADS;
__global__ void __launch_bounds__(kIadDcThreads, 1) iad_dc_kernel(Fields F, Params P) {
  const int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (i >= F.n) return;
  const Geom g = load_geom(F.ds, P);
  const Rec4 me = F.rec_i[i];
  if (is_ghost(F, i)) {
    if (P.part != SPH_PART_INTERIOR) ghost_rec_m(F, i, me);
    return;
  }
  if (!in_part(F, P.part, i)) return;
  if (__any_sync(__activemask(), needs_wrap(g, me.a, me.b, me.c, F.f[FH][i])))
    iad_dc_body<true>(F, P, g, i, me);
  else
    iad_dc_body<false>(F, P, g, i, me);
}

__global__ void __launch_bounds__(kIadThreads, 768 / kIadThreads) iad_kernel(Fields F, Params P) {
  const int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (i >= F.n) return;
  const Geom g = load_geom(F.ds, P);
  const Rec4 me = F.rec_i[i];
  if (is_ghost(F, i)) {
    if (P.part != SPH_PART_INTERIOR) ghost_rec_m(F, i, me);
    return;
  }
  if (!in_part(F, P.part, i)) return;
  if (__any_sync(__activemask(), needs_wrap(g, me.a, me.b, me.c, F.f[FH][i])))
    iad_body<true>(F, g, i, me);
  else
    iad_body<false>(F, g, i, me);
}

// ------------------------------------------------------------------ momentum-energy
// a_i = -sum_j m_j [(p_i/rho_i^2) A + (p_j/rho_j^2) B + Pi G],
// du_i = sum_j m_j [(p_i/rho_i^2) v_ij.A + Pi/2 v_ij.G],
// A = C_i Delta W(r,h_i), B = C_j Delta W(r,h_j), G = (A+B)/2, Monaghan Pi.
// Also the warp-min of h_i/c_i for the time step (exact: integer atomicMin on the
// order-preserving bit pattern of a positive double).
// Per pair: 4 records (128 B) + 1 more (AV) for approaching pairs, 157 DP flops
// (+ 17 and 2 divisions when approaching).
template <bool kWrap, bool kSwitch, bool kVsig>
__device__ __forceinline__ double momentum_body(const Fields& F, const Params& P, const Geom& g, int64_t i) {
  const Rec4* __restrict__ rec = F.rec_m;
  const Rec4* mi = rec + (int64_t)kRecM * i;
  const Rec4 i0 = mi[0], i1 = mi[1], i2 = mi[2], i3 = mi[3], i4 = mi[4];
  const double xi = i0.a, yi = i0.b, zi = i0.c, qi = i0.d;
  const double ci11 = i1.a, ci12 = i1.b, ci13 = i1.c, khi = i1.d;
  const double ci22 = i2.a, ci23 = i2.b, ci33 = i2.c;
  const double vxi = i3.a, vyi = i3.b, vzi = i3.c, pri = i3.d;
  const double hi = i4.a, ci = i4.b, rhoi = i4.c, fi = i4.d;
  const double alpha = P.av_alpha, beta = P.av_beta, eps = P.av_eps;
  const int nci = min(F.nc[i], F.ngmax);
  double ax = 0, ay = 0, az = 0, de = 0;
  double vs = kVsig ? 2.0 * ci : ci;  // signal velocity (reading 22); c_i without it
  const int32_t* __restrict__ nb = F.nbr + i;
  // software pipeline: neighbour index three ahead, the position chunk (needed
  // first) two ahead; the other chunks are loaded at the top of the iteration
  // and arrive while the two sinc polynomials run.
  const int64_t cap = F.cap;
  const Rec4* r0 = rec + (int64_t)kRecM * (nci > 0 ? ldg_idx(nb) : 0);
  const Rec4* r1 = rec + (int64_t)kRecM * (nci > 1 ? ldg_idx(nb + cap) : 0);
  int jn = nci > 2 ? ldg_idx(nb + 2 * cap) : 0;
  Rec4 p0 = ldg4(r0), p1 = ldg4(r1);
  for (int k = 0; k < nci; ++k) {
    const Rec4* rcur = r0;
    const Rec4 j1 = ldg4(rcur + 1), j2 = ldg4(rcur + 2), j3 = ldg4(rcur + 3);
    const Rec4 j0 = p0;
    p0 = p1;
    r0 = r1;
    if (k + 2 < nci) {
#if SPH_MOM_DIAG == 2
      r1 = rec + (int64_t)kRecM * ((i & ~31ll) + ((jn & 1) ? 1 : 0));  // diagnostic: broadcast records
#else
      r1 = rec + (int64_t)kRecM * jn;
#endif
      p1 = ldg4(r1);
    }
    if (k + 3 < nci) jn = ldg_idx(nb + (int64_t)(k + 3) * cap);
#if SPH_MOM_DIAG == 1
    // diagnostic: the gathers alone (every load, no pair arithmetic)
    ax += j0.a + j1.a + j2.b + j3.c;
    if (j0.d < 0.0) {  // never: keeps the AV-chunk load of ~half the pairs
      const Rec4 j4d = ldg4(rcur + 4);
      ay += j4d.a;
    }
    if ((k & 1) == 0) {
      const Rec4 j4d = ldg4(rcur + 4);
      az += j4d.b;
    }
    continue;
#endif
    double dx, dy, dz;
    pair_d<kWrap>(g, xi, yi, zi, j0.a, j0.b, j0.c, dx, dy, dz);
    const double r2 = dx * dx + dy * dy + dz * dz;
    const double wi = khi * sinc6_t_cb(r2 * qi);
    const double tj = r2 * j0.d;
    const double wj = tj < kPi2 ? j1.d * sinc6_t_cb(tj) : 0.0;
    // Delta = -d.  With A = w_i C_i Delta, B = w_j C_j Delta, G = (A+B)/2 the
    // pair terms regroup exactly (up to rounding) as
    //   (p_i/rho_i^2) A + (p_j/rho_j^2) B + Pi G
    //     = (p_i/rho_i^2 + Pi/2) w_i C_i Delta + (p_j/rho_j^2 + Pi/2) w_j C_j Delta,
    //   (p_i/rho_i^2) v.A + Pi/2 v.G
    //     = (p_i/rho_i^2 + Pi/4) w_i v.C_i Delta + (Pi/4) w_j v.C_j Delta,
    // which saves the scaled vectors A, B, G (~9 DP instructions per pair).
    const double Dx = -dx, Dy = -dy, Dz = -dz;
    const double CiDx = ci11 * Dx + ci12 * Dy + ci13 * Dz;
    const double CiDy = ci12 * Dx + ci22 * Dy + ci23 * Dz;
    const double CiDz = ci13 * Dx + ci23 * Dy + ci33 * Dz;
    const double CjDx = j1.a * Dx + j1.b * Dy + j1.c * Dz;
    const double CjDy = j1.b * Dx + j2.a * Dy + j2.b * Dz;
    const double CjDz = j1.c * Dx + j2.b * Dy + j2.c * Dz;
    const double vx = vxi - j3.a, vy = vyi - j3.b, vz = vzi - j3.c;
    const double rv = dx * vx + dy * vy + dz * vz;
    double Pi = 0.0;
    Rec4 j4v;
    if (kVsig) {  // vsig_ij = c_i + c_j - 3 min(0, rv / r)
      j4v = ldg4(rcur + 4);
      const double w = rv < 0.0 ? rv * rsqrt(r2) : 0.0;
      vs = fmax(vs, ci + j4v.b - 3.0 * w);
    }
    {
      // branch-free AV: the AV chunk is loaded by approaching lanes only (a
      // predicated load; receding lanes use their own values, finite), Pi is
      // formed by every lane and zeroed for receding pairs
      Rec4 j4;
      if (kVsig) j4 = j4v; else { j4.a = hi; j4.b = ci; j4.c = rhoi; j4.d = fi; }
      if (!kVsig && rv < 0.0) j4 = ldg4(rcur + 4);
      const double hbar = 0.5 * (hi + j4.a);
      const double cbar = 0.5 * (ci + j4.b);
      const double rhobar = 0.5 * (rhoi + j4.c);
      const double D = fma(eps * hbar, hbar, r2);
      const double q = 1.0 / (D * rhobar);
      const double mu = hbar * rv * (rhobar * q);
      double pv = (fma(beta, mu, -alpha * cbar) * mu) * (D * q);
      if (kSwitch) pv *= 0.5 * (fi + j4.d);
      Pi = rv < 0.0 ? pv : 0.0;
    }
    const double mj = j2.d, prj = j3.d;
    const double ka = (pri + 0.5 * Pi) * wi, kb = (prj + 0.5 * Pi) * wj;
    ax -= mj * fma(ka, CiDx, kb * CjDx);
    ay -= mj * fma(ka, CiDy, kb * CjDy);
    az -= mj * fma(ka, CiDz, kb * CjDz);
    const double vCi = vx * CiDx + vy * CiDy + vz * CiDz;
    const double vCj = vx * CjDx + vy * CjDy + vz * CjDz;
    de += mj * fma((pri + 0.25 * Pi) * wi, vCi, 0.25 * Pi * wj * vCj);
  }
  F.ax[i] = ax;
  F.ay[i] = ay;
  F.az[i] = az;
  F.du[i] = de;
  if (kVsig) F.vsig[i] = vs;
  return vs;
}

__global__ void __launch_bounds__(kMomThreads, kMomThreads >= 512 ? 1 : 512 / kMomThreads) momentum_energy_kernel(Fields F, Params P) {
  const int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  // ghosts: no sums, not in the dt minimum; a split launch takes its class only
  const bool active = i < F.n && !is_ghost(F, i) && in_part(F, P.part, i);
  unsigned long long hc = ~0ull;
  if (active) {
    const Geom g = load_geom(F.ds, P);
    const Rec4* mi = F.rec_m + (int64_t)kRecM * i;
    const Rec4 i0 = mi[0], i4 = mi[4];
    const bool wrap = __any_sync(__activemask(), needs_wrap(g, i0.a, i0.b, i0.c, i4.a));
    double vs;  // c_i, or the signal velocity with cfg.dt_vsig
    if (P.dt_vsig) {
      if (P.av_switch) vs = wrap ? momentum_body<true, true, true>(F, P, g, i) : momentum_body<false, true, true>(F, P, g, i);
      else vs = wrap ? momentum_body<true, false, true>(F, P, g, i) : momentum_body<false, false, true>(F, P, g, i);
    } else if (P.av_switch) {
      vs = wrap ? momentum_body<true, true, false>(F, P, g, i) : momentum_body<false, true, false>(F, P, g, i);
    } else {
      vs = wrap ? momentum_body<true, false, false>(F, P, g, i) : momentum_body<false, false, false>(F, P, g, i);
    }
    hc = ord_of(__ddiv_rn(i4.a, vs));
  }
#pragma unroll
  for (int off = 16; off > 0; off >>= 1) {
    unsigned long long t = __shfl_xor_sync(0xffffffffu, hc, off);
    hc = t < hc ? t : hc;
  }
  if ((threadIdx.x & 31) == 0 && hc != ~0ull) atomicMin(&F.ds->minhc_ord, hc);
}

// ------------------------------------------------------------------ time step
// dt = min(C * min_i h_i/c_i, growth * dt_prev)  (same operations as the oracle).
__global__ void timestep_kernel(DevScalars* ds, Params P) {
  double mhc = ds->minhc_ord == ~0ull ? INFINITY : unord(ds->minhc_ord);
  double a = __dmul_rn(P.k_cour, mhc), b = __dmul_rn(P.dt_max_growth, ds->dt_prev);
  ds->dt = a < b ? a : b;
}

// ------------------------------------------------------------------ update
// Item 10: kick (v at half steps), drift + periodic wrap, AB2 energy, h update.
// HBM-bound: 13 doubles + nc read, 9 doubles written per particle.
__global__ void __launch_bounds__(256) update_kernel(Fields F, Params P) {
  const int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (i >= F.n) return;
  const DevScalars* ds = F.ds;
  const double dt = ds->dt, dtm1 = ds->dt_prev;
  const int first = ds->first;
  const double acc[3] = {F.ax[i], F.ay[i], F.az[i]};
#pragma unroll
  for (int a = 0; a < 3; ++a) {
    double v = F.f[FVX + a][i] + acc[a] * (dt + dtm1) / 2.0;
    double x = F.f[FX + a][i] + v * dt;
    if (P.periodic[a]) {
      const double lo = ds->box_min[a], hi = ds->box_max[a], L = hi - lo;
      if (x >= hi) x -= L;
      else if (x < lo) x += L;
    }
    F.f[FVX + a][i] = v;
    F.f[FX + a][i] = x;
  }
  const double du = F.du[i];
  const double dum1 = first ? du : F.f[FDUM1][i];
  const double half = dt * dt / (2.0 * dtm1);
  F.f[FU][i] = F.f[FU][i] + du * (dt + half) - dum1 * half;
  F.f[FDUM1][i] = du;
  const int nc = F.nc[i];
  const double ncd = nc > 1 ? (double)nc : 1.0;
  const double hn = F.f[FH][i] * 0.5 * pow(1.0 + 1023.0 * P.ng0 / ncd, 0.1);
  F.f[FH][i] = hn < P.h_cap ? hn : P.h_cap;
}

__global__ void advance_time_kernel(DevScalars* ds) {
  ds->t += ds->dt;
  ds->dt_prev = ds->dt;
  ds->first = 0;
}

// Rebuilds the C chunks of the momentum records after sph_set_field wrote the
// owners' C over the ghosts (multi-GPU halo, item 8(e)).
__global__ void __launch_bounds__(256) refresh_rec_m_kernel(Fields F) {
  const int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (i >= F.n) return;
  Rec4* rm = F.rec_m + (int64_t)kRecM * i;
  st4(rm + 1, F.C[0][i], F.C[1][i], F.C[2][i], F.wk[i]);
  st4(rm + 2, F.C[3][i], F.C[4][i], F.C[5][i], F.f[FM][i]);
  if (F.bal) rm[4].d = F.bal[i];  // owners' Balsara factors over the ghosts (av_switch)
}

void launch_refresh_rec_m(const Fields& F, cudaStream_t st) {
  if (F.n == 0) return;
  refresh_rec_m_kernel<<<(unsigned)div_up(F.n, 256), 256, 0, st>>>(F);
  note_launch();
}

// ------------------------------------------------------------------ launchers
void launch_density(const Fields& F, const Params& P, cudaStream_t st) {
  if (F.n == 0) return;
  density_kernel<<<(unsigned)div_up(F.n, kDensThreads), kDensThreads, 0, st>>>(F, P);
  note_launch();
}
void launch_eos(const Fields& F, const Params& P, cudaStream_t st, bool apply_omega) {
  if (F.n == 0) return;
  eos_kernel<<<(unsigned)div_up(F.n, 256), 256, 0, st>>>(F, P, apply_omega);
  note_launch();
}
void launch_iad(const Fields& F, const Params& P, cudaStream_t st) {
  if (F.n == 0) return;
  if (P.divcurl)
    iad_dc_kernel<<<(unsigned)div_up(F.n, kIadDcThreads), kIadDcThreads, 0, st>>>(F, P);
  else
    iad_kernel<<<(unsigned)div_up(F.n, kIadThreads), kIadThreads, 0, st>>>(F, P);
  note_launch();
}
void launch_gradh(const Fields& F, const Params& P, cudaStream_t st) {
  if (F.n == 0) return;
  gradh_kernel<<<(unsigned)div_up(F.n, kDensThreads), kDensThreads, 0, st>>>(F, P);
  note_launch();
}
void launch_prho2(const Fields& F, cudaStream_t st) {
  if (F.n == 0) return;
  prho2_kernel<<<(unsigned)div_up(F.n, 256), 256, 0, st>>>(F);
  note_launch();
}
void launch_momentum_energy(const Fields& F, const Params& P, cudaStream_t st) {
  if (F.n == 0) return;
  momentum_energy_kernel<<<(unsigned)div_up(F.n, kMomThreads), kMomThreads, 0, st>>>(F, P);
  note_launch();
}
void launch_timestep(const Fields& F, const Params& P, cudaStream_t st) {
  timestep_kernel<<<1, 1, 0, st>>>(F.ds, P);
  note_launch();
}
void launch_update(const Fields& F, const Params& P, cudaStream_t st) {
  if (F.n == 0) return;
  update_kernel<<<(unsigned)div_up(F.n, 256), 256, 0, st>>>(F, P);
  note_launch();
}
void launch_advance_time(const Fields& F, cudaStream_t st) {
  advance_time_kernel<<<1, 1, 0, st>>>(F.ds);
  note_launch();
}

}  // namespace sph
