// k_physics.cu -- phases DENSITY, EOS, IAD, MOMENTUM_ENERGY, TIMESTEP, UPDATE
// (items 5-10 of DESIGN.md section 3; the paper's XMass P:184,
// IADVelocityDivCurl P:180, MomentumEnergy P:160/P:180, the end-of-step
// collective P:220).
//
// The three neighbour sums run one thread per target over its stored list in
// list order (ascending j, the oracle's summation order).  Lists are column-
// major so the k-th neighbour indices of a warp's 32 consecutive targets are
// one coalesced 128-B load; the j-side fields are gathers that hit L1/L2
// because consecutive targets share most neighbours (Morton order).  The sinc
// kernel is a polynomial in t = r^2 (pi/2h)^2 (no sqrt/sin per pair); the
// per-particle factors (pi/2h)^2 and K/h^3 are computed once per particle by the
// density kernel.  All of them are FP64-bound.
#include <algorithm>

#include "sph_internal.cuh"

namespace sph {

constexpr double kPi = 3.14159265358979323846;
constexpr double kPi2Over4 = kPi * kPi / 4.0;
constexpr double kPi2 = kPi * kPi;

struct Geom {
  double L[3], H[3];
  bool per[3];
};

__device__ __forceinline__ Geom load_geom(const DevScalars* ds, const Params& P) {
  Geom g;
#pragma unroll
  for (int a = 0; a < 3; ++a) {
    g.L[a] = ds->box_max[a] - ds->box_min[a];
    g.H[a] = 0.5 * g.L[a];
    g.per[a] = P.periodic[a] != 0;
  }
  return g;
}

// ------------------------------------------------------------------ density
// rho_i = (K/h_i^3) [m_i + sum_j m_j S(pi r_ij / 2h_i)^6]; also writes the
// per-particle kernel factors wq = (pi/2h)^2 and wk = K/h^3 reused by IAD and
// momentum-energy.  Per pair: 4 gathered doubles (x, y, z, m), ~27 DP flops.
__global__ void __launch_bounds__(256) density_kernel(Fields F, Params P, double* __restrict__ wq,
                                                      double* __restrict__ wk) {
  const int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (i >= F.n) return;
  const Geom g = load_geom(F.ds, P);
  const double* __restrict__ X = F.f[FX];
  const double* __restrict__ Y = F.f[FY];
  const double* __restrict__ Z = F.f[FZ];
  const double* __restrict__ M = F.f[FM];
  const double xi = X[i], yi = Y[i], zi = Z[i], hi = F.f[FH][i];
  const double q = kPi2Over4 / (hi * hi);
  const double kh3 = P.K / (hi * hi * hi);
  const int nci = min(F.nc[i], F.ngmax);
  double sum = M[i];
  const int32_t* __restrict__ nb = F.nbr + i;
  for (int k = 0; k < nci; ++k) {
    const int j = __ldg(nb + (int64_t)k * F.cap);
    double dx = min_image(xi - __ldg(X + j), g.L[0], g.H[0], g.per[0]);
    double dy = min_image(yi - __ldg(Y + j), g.L[1], g.H[1], g.per[1]);
    double dz = min_image(zi - __ldg(Z + j), g.L[2], g.H[2], g.per[2]);
    double r2 = dx * dx + dy * dy + dz * dz;
    sum = fma(__ldg(M + j), sinc6_t(r2 * q), sum);
  }
  F.rho[i] = kh3 * sum;
  wq[i] = q;
  wk[i] = kh3;
}

// ------------------------------------------------------------------ EOS
// Bit-exact vs the oracle (same operation order, IEEE sqrt/div): p, c, and the
// derived per-particle V = m/rho and p/rho^2 used by the next two sums.
__global__ void __launch_bounds__(256) eos_kernel(Fields F, Params P) {
  const int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (i >= F.n) return;
  const double rho = F.rho[i], u = F.f[FU][i];
  double p, c;
  if (P.eos == SPH_EOS_IDEAL) {
    p = __dmul_rn(__dmul_rn(P.gamma - 1.0, rho), u);
    c = __dsqrt_rn(__dmul_rn(__dmul_rn(P.gamma, P.gamma - 1.0), u));
  } else {
    p = __dmul_rn(__dmul_rn(P.cs0, P.cs0), rho);
    c = P.cs0;
  }
  F.p[i] = p;
  F.c[i] = c;
  F.vol[i] = __ddiv_rn(F.f[FM][i], rho);
  F.prho2[i] = __ddiv_rn(p, __dmul_rn(rho, rho));
}

// ------------------------------------------------------------------ IAD
// tau_i = sum_j V_j W(r,h_i) Delta Delta^T, C_i = tau_i^{-1} (adjugate / det).
// Per pair: 4 gathered doubles (x, y, z, V), ~41 DP flops.
__global__ void __launch_bounds__(256) iad_kernel(Fields F, Params P, const double* __restrict__ wq,
                                                  const double* __restrict__ wk) {
  const int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (i >= F.n) return;
  const Geom g = load_geom(F.ds, P);
  const double* __restrict__ X = F.f[FX];
  const double* __restrict__ Y = F.f[FY];
  const double* __restrict__ Z = F.f[FZ];
  const double* __restrict__ V = F.vol;
  const double xi = X[i], yi = Y[i], zi = Z[i];
  const double q = wq[i], kh3 = wk[i];
  const int nci = min(F.nc[i], F.ngmax);
  double t11 = 0, t12 = 0, t13 = 0, t22 = 0, t23 = 0, t33 = 0;
  const int32_t* __restrict__ nb = F.nbr + i;
  for (int k = 0; k < nci; ++k) {
    const int j = __ldg(nb + (int64_t)k * F.cap);
    double dx = min_image(xi - __ldg(X + j), g.L[0], g.H[0], g.per[0]);
    double dy = min_image(yi - __ldg(Y + j), g.L[1], g.H[1], g.per[1]);
    double dz = min_image(zi - __ldg(Z + j), g.L[2], g.H[2], g.per[2]);
    double r2 = dx * dx + dy * dy + dz * dz;
    double vw = __ldg(V + j) * (kh3 * sinc6_t(r2 * q));
    // Delta = -d; the products Delta^a Delta^b equal d^a d^b.
    double ax = vw * dx, ay = vw * dy, az = vw * dz;
    t11 = fma(ax, dx, t11);
    t12 = fma(ax, dy, t12);
    t13 = fma(ax, dz, t13);
    t22 = fma(ay, dy, t22);
    t23 = fma(ay, dz, t23);
    t33 = fma(az, dz, t33);
  }
  const double det = t11 * (t22 * t33 - t23 * t23) - t12 * (t12 * t33 - t23 * t13) +
                     t13 * (t12 * t23 - t22 * t13);
  const double inv = 1.0 / det;
  F.C[0][i] = (t22 * t33 - t23 * t23) * inv;
  F.C[1][i] = (t13 * t23 - t12 * t33) * inv;
  F.C[2][i] = (t12 * t23 - t13 * t22) * inv;
  F.C[3][i] = (t11 * t33 - t13 * t13) * inv;
  F.C[4][i] = (t12 * t13 - t11 * t23) * inv;
  F.C[5][i] = (t11 * t22 - t12 * t12) * inv;
  if (!(det > 0.0) || !isfinite(det)) atomicOr(&F.ds->status, (int)ST_SINGULAR);
}

// ------------------------------------------------------------------ momentum-energy
// a_i = -sum_j m_j [(p_i/rho_i^2) A + (p_j/rho_j^2) B + Pi G],
// du_i = sum_j m_j [(p_i/rho_i^2) v_ij.A + Pi/2 v_ij.G],
// A = C_i Delta W(r,h_i), B = C_j Delta W(r,h_j), G = (A+B)/2, Monaghan Pi.
// Also the warp-min of h_i/c_i for the time step (exact: integer atomicMin on the
// order-preserving bit pattern of a positive double).
// Per pair: 18 gathered doubles, ~150 DP flops (+ 2 divisions when approaching).
__global__ void __launch_bounds__(128) momentum_energy_kernel(Fields F, Params P,
                                                              const double* __restrict__ wq,
                                                              const double* __restrict__ wk) {
  const int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  const bool active = i < F.n;
  unsigned long long hc = ~0ull;
  if (active) {
    const Geom g = load_geom(F.ds, P);
    const double* __restrict__ X = F.f[FX];
    const double* __restrict__ Y = F.f[FY];
    const double* __restrict__ Z = F.f[FZ];
    const double* __restrict__ VX = F.f[FVX];
    const double* __restrict__ VY = F.f[FVY];
    const double* __restrict__ VZ = F.f[FVZ];
    const double* __restrict__ Hh = F.f[FH];
    const double* __restrict__ M = F.f[FM];
    const double* __restrict__ RHO = F.rho;
    const double* __restrict__ PR = F.prho2;
    const double* __restrict__ CS = F.c;
    const double* __restrict__ C0 = F.C[0];
    const double* __restrict__ C1 = F.C[1];
    const double* __restrict__ C2 = F.C[2];
    const double* __restrict__ C3 = F.C[3];
    const double* __restrict__ C4 = F.C[4];
    const double* __restrict__ C5 = F.C[5];
    const double xi = X[i], yi = Y[i], zi = Z[i];
    const double vxi = VX[i], vyi = VY[i], vzi = VZ[i];
    const double hi = Hh[i], rhoi = RHO[i], pri = PR[i], ci = CS[i];
    const double ci11 = C0[i], ci12 = C1[i], ci13 = C2[i], ci22 = C3[i], ci23 = C4[i], ci33 = C5[i];
    const double qi = wq[i], khi = wk[i];
    const double alpha = P.av_alpha, beta = P.av_beta, eps = P.av_eps;
    const int nci = min(F.nc[i], F.ngmax);
    double ax = 0, ay = 0, az = 0, de = 0;
    const int32_t* __restrict__ nb = F.nbr + i;
    for (int k = 0; k < nci; ++k) {
      const int j = __ldg(nb + (int64_t)k * F.cap);
      const double dx = min_image(xi - __ldg(X + j), g.L[0], g.H[0], g.per[0]);
      const double dy = min_image(yi - __ldg(Y + j), g.L[1], g.H[1], g.per[1]);
      const double dz = min_image(zi - __ldg(Z + j), g.L[2], g.H[2], g.per[2]);
      const double r2 = dx * dx + dy * dy + dz * dz;
      const double wi = khi * sinc6_t(r2 * qi);
      const double tj = r2 * __ldg(wq + j);
      const double wj = tj < kPi2 ? __ldg(wk + j) * sinc6_t(tj) : 0.0;
      // Delta = -d
      const double Dx = -dx, Dy = -dy, Dz = -dz;
      const double cj11 = __ldg(C0 + j), cj12 = __ldg(C1 + j), cj13 = __ldg(C2 + j);
      const double cj22 = __ldg(C3 + j), cj23 = __ldg(C4 + j), cj33 = __ldg(C5 + j);
      const double Ax = (ci11 * Dx + ci12 * Dy + ci13 * Dz) * wi;
      const double Ay = (ci12 * Dx + ci22 * Dy + ci23 * Dz) * wi;
      const double Az = (ci13 * Dx + ci23 * Dy + ci33 * Dz) * wi;
      const double Bx = (cj11 * Dx + cj12 * Dy + cj13 * Dz) * wj;
      const double By = (cj12 * Dx + cj22 * Dy + cj23 * Dz) * wj;
      const double Bz = (cj13 * Dx + cj23 * Dy + cj33 * Dz) * wj;
      const double Gx = 0.5 * (Ax + Bx), Gy = 0.5 * (Ay + By), Gz = 0.5 * (Az + Bz);
      const double vx = vxi - __ldg(VX + j), vy = vyi - __ldg(VY + j), vz = vzi - __ldg(VZ + j);
      const double rv = dx * vx + dy * vy + dz * vz;
      double Pi = 0.0;
      if (rv < 0.0) {
        const double hbar = 0.5 * (hi + __ldg(Hh + j));
        const double cbar = 0.5 * (ci + __ldg(CS + j));
        const double rhobar = 0.5 * (rhoi + __ldg(RHO + j));
        const double mu = hbar * rv / (r2 + eps * hbar * hbar);
        Pi = (-alpha * cbar * mu + beta * mu * mu) / rhobar;
      }
      const double mj = __ldg(M + j), prj = __ldg(PR + j);
      ax -= mj * (pri * Ax + prj * Bx + Pi * Gx);
      ay -= mj * (pri * Ay + prj * By + Pi * Gy);
      az -= mj * (pri * Az + prj * Bz + Pi * Gz);
      de += mj * (pri * (vx * Ax + vy * Ay + vz * Az) + 0.5 * Pi * (vx * Gx + vy * Gy + vz * Gz));
    }
    F.ax[i] = ax;
    F.ay[i] = ay;
    F.az[i] = az;
    F.du[i] = de;
    hc = ord_of(__ddiv_rn(hi, ci));
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

// ------------------------------------------------------------------ launchers
void launch_density(const Fields& F, const Params& P, cudaStream_t st) {
  if (F.n == 0) return;
  density_kernel<<<(unsigned)div_up(F.n, 256), 256, 0, st>>>(F, P, F.wq, F.wk); note_launch();
}
void launch_eos(const Fields& F, const Params& P, cudaStream_t st) {
  if (F.n == 0) return;
  eos_kernel<<<(unsigned)div_up(F.n, 256), 256, 0, st>>>(F, P); note_launch();
}
void launch_iad(const Fields& F, const Params& P, cudaStream_t st) {
  if (F.n == 0) return;
  iad_kernel<<<(unsigned)div_up(F.n, 256), 256, 0, st>>>(F, P, F.wq, F.wk); note_launch();
}
void launch_momentum_energy(const Fields& F, const Params& P, cudaStream_t st) {
  if (F.n == 0) return;
  momentum_energy_kernel<<<(unsigned)div_up(F.n, 128), 128, 0, st>>>(F, P, F.wq, F.wk); note_launch();
}
void launch_timestep(const Fields& F, const Params& P, cudaStream_t st) {
  timestep_kernel<<<1, 1, 0, st>>>(F.ds, P); note_launch();
}
void launch_update(const Fields& F, const Params& P, cudaStream_t st) {
  if (F.n == 0) return;
  update_kernel<<<(unsigned)div_up(F.n, 256), 256, 0, st>>>(F, P); note_launch();
}
void launch_advance_time(const Fields& F, cudaStream_t st) { advance_time_kernel<<<1, 1, 0, st>>>(F.ds); note_launch(); }

}  // namespace sph
