// k_stir.cu -- phase STIR: Ornstein-Uhlenbeck turbulence driving (
// the Subsonic Turbulence workload of P:108; definitions in include/sph.h).
//
// Two kernels per step:
//  * stir_ou_kernel (1 CTA, one thread per mode): A <- f A + sigma sqrt(1-f^2) xi_s
//    with f = exp(-dt_prev/t_decay), then the Helmholtz projection
//    A^ = zeta A_perp + (1-zeta) A_par = zeta A + (1 - 2 zeta) k^(k^.A) and
//    B = 2 w A^ (the factor 2 folds the -n partner of each half-space mode);
//  * stir_accel_kernel (one thread per particle): a_i += sum_m Re(B_m e^{i k_m.(x_i-lo)}).
//    e^{i k.x} = prod_a (e^{i theta_a})^{n_a}: one sincos per axis (theta_a =
//    2 pi (x_a - lo_a)/L_a) and complex products for the powers |n_a| <= 3, so a
//    mode costs one complex multiply (4 DP ops) and six FMAs instead of a
//    sin/cos pair.  The mode loop is fully unrolled over the fixed set (n_x 0..3,
//    n_y, n_z -3..3, half space, 1 <= |n|^2 <= 9): all power-table indices are
//    compile-time, the B coefficients are broadcast reads from shared memory.
// Bound: FP64 (~700 DP instructions per particle), 24 B read + 24 B read/written.
#include "sph_internal.cuh"

namespace sph {

constexpr double kTwoPi = 6.283185307179586476925286766559;

__host__ __device__ constexpr bool half_space(int nx, int ny, int nz) {
  return nx > 0 || (nx == 0 && (ny > 0 || (ny == 0 && nz > 0)));
}
__host__ __device__ constexpr bool in_set(int nx, int ny, int nz) {
  return half_space(nx, ny, nz) && nx * nx + ny * ny + nz * nz >= 1 && nx * nx + ny * ny + nz * nz <= 9;
}

int stir_modes(int32_t* n3) {
  int m = 0;
  for (int nx = 0; nx <= 3; ++nx)
    for (int ny = -3; ny <= 3; ++ny)
      for (int nz = -3; nz <= 3; ++nz)
        if (in_set(nx, ny, nz)) {
          if (n3) {
            n3[3 * m] = nx;
            n3[3 * m + 1] = ny;
            n3[3 * m + 2] = nz;
          }
          ++m;
        }
  return m;
}

__constant__ int c_modes[kStirModes][3];

__global__ void stir_ou_kernel(DevScalars* ds, Stir S, double Lx, double Ly, double Lz) {
  const int m = threadIdx.x;
  const unsigned long long step = ds->stir_step;
  if (step >= (unsigned long long)S.nsteps) {  // noise table exhausted
    if (m == 0) atomicOr(&ds->status, (int)ST_STIR_NOISE);
    return;
  }
  if (m < kStirModes) {
    const double f = exp(-ds->dt_prev / S.t_decay);
    const double g = S.sigma * sqrt(1.0 - f * f);
    const double* xi = S.noise + ((size_t)step * kStirModes + m) * 6;
    double a[6];
#pragma unroll
    for (int c = 0; c < 6; ++c) {
      a[c] = f * S.A[m * 6 + c] + g * xi[c];
      S.A[m * 6 + c] = a[c];
    }
    // unit wave vector (k_a = 2 pi n_a / L_a; 2 pi cancels)
    const double kx = c_modes[m][0] / Lx, ky = c_modes[m][1] / Ly, kz = c_modes[m][2] / Lz;
    const double kn = sqrt(kx * kx + ky * ky + kz * kz);
    const double ux = kx / kn, uy = ky / kn, uz = kz / kn;
    const double s = 2.0 * S.w[m], z = S.zeta;
#pragma unroll
    for (int part = 0; part < 2; ++part) {  // real, imaginary
      const double vx = a[0 + part], vy = a[2 + part], vz = a[4 + part];
      const double kv = (1.0 - 2.0 * z) * (ux * vx + uy * vy + uz * vz);
      S.B[m * 6 + 0 + part] = s * (z * vx + kv * ux);
      S.B[m * 6 + 2 + part] = s * (z * vy + kv * uy);
      S.B[m * 6 + 4 + part] = s * (z * vz + kv * uz);
    }
  }
  __syncthreads();
  if (m == 0) ds->stir_step = step + 1;
}

struct Cx {
  double re, im;
};
__device__ __forceinline__ Cx cmul(Cx a, Cx b) { return {fma(a.re, b.re, -a.im * b.im), fma(a.re, b.im, a.im * b.re)}; }
__device__ __forceinline__ Cx cpow_n(const Cx (&p)[4], int n) {  // e^{i n theta}, |n| <= 3
  const Cx v = p[n < 0 ? -n : n];
  return n < 0 ? Cx{v.re, -v.im} : v;
}

__global__ void __launch_bounds__(256) stir_accel_kernel(Fields F, Stir S) {
  __shared__ double sB[kStirModes * 6];
  for (int k = threadIdx.x; k < kStirModes * 6; k += blockDim.x) sB[k] = S.B[k];
  __syncthreads();
  const int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (i >= F.n) return;
  const DevScalars* ds = F.ds;
  if (ds->status & ST_STIR_NOISE) return;
  Cx P[3][4];
#pragma unroll
  for (int a = 0; a < 3; ++a) {
    const double lo = ds->box_min[a], L = ds->box_max[a] - lo;
    double sn, cs;
    sincos(kTwoPi * ((F.f[FX + a][i] - lo) / L), &sn, &cs);
    P[a][0] = {1.0, 0.0};
    P[a][1] = {cs, sn};
    P[a][2] = cmul(P[a][1], P[a][1]);
    P[a][3] = cmul(P[a][2], P[a][1]);
  }
  double ax = 0.0, ay = 0.0, az = 0.0;
  int m = 0;
#pragma unroll
  for (int nx = 0; nx <= 3; ++nx) {
#pragma unroll
    for (int ny = -3; ny <= 3; ++ny) {
      const Cx q = cmul(P[0][nx], cpow_n(P[1], ny));
#pragma unroll
      for (int nz = -3; nz <= 3; ++nz) {
        if (in_set(nx, ny, nz)) {
          const Cx e = cmul(q, cpow_n(P[2], nz));
          const double* b = sB + 6 * m;
          ax = fma(b[0], e.re, fma(-b[1], e.im, ax));
          ay = fma(b[2], e.re, fma(-b[3], e.im, ay));
          az = fma(b[4], e.re, fma(-b[5], e.im, az));
          ++m;
        }
      }
    }
  }
  F.ax[i] += ax;
  F.ay[i] += ay;
  F.az[i] += az;
}

// The mode table in constant memory; called by sph_stir_init (a synchronous
// copy: never inside a captured step graph).
void stir_upload_modes() {
  static bool modes_set = false;
  if (!modes_set) {
    int32_t n3[3 * kStirModes];
    stir_modes(n3);
    cudaMemcpyToSymbol(c_modes, n3, sizeof(n3));
    modes_set = true;
  }
}

void launch_stir(const Fields& F, const Params& P, const Stir& S, cudaStream_t st) {
  stir_upload_modes();  // no-op after sph_stir_init
  (void)P;
  // the box lengths of periodic axes are the configured ones (stirring is for
  // periodic boxes; open axes use the step's box)
  stir_ou_kernel<<<1, 64, 0, st>>>(F.ds, S, P.box_max[0] - P.box_min[0], P.box_max[1] - P.box_min[1],
                                   P.box_max[2] - P.box_min[2]);
  note_launch();
  if (F.n > 0) {
    stir_accel_kernel<<<(unsigned)div_up(F.n, 256), 256, 0, st>>>(F, S);
    note_launch();
  }
}

}  // namespace sph
