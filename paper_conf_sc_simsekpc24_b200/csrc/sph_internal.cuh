// sph_internal.cuh -- private types and device helpers of libsph.
//
// Layout of the data in HBM: every per-particle field is
// a separate fp64 (or int) array of n_capacity entries inside the caller's arena
// (structure of arrays, coalesced per field).  Persistent particle state is
// double-buffered so that the sort's permutation gathers from one buffer into
// the other.  Neighbour lists are stored column-major, nbr[k * cap + i], so that
// a warp of 32 consecutive targets reads its k-th neighbours in one 128-B line.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include <atomic>

#include "../../include/sph.h"

namespace sph {

constexpr int kNumStateF = 10;  // x y z vx vy vz h m u du_m1 (fp64) + id (int64)
enum StateField { FX = 0, FY, FZ, FVX, FVY, FVZ, FH, FM, FU, FDUM1 };

// Onesweep radix sort geometry (k_sort.cu).
constexpr int kSortThreads = 256;
#ifndef SPH_SORT_KPT
#define SPH_SORT_KPT 8  // keys per thread (A/B builds)
#endif
constexpr int kSortKPT = SPH_SORT_KPT;
constexpr int kSortTile = kSortThreads * kSortKPT;  // 2048 keys per tile (4 CTAs/SM, SPH_SORT_MINB)
constexpr int kRadixBits = 8;
constexpr int kRadix = 256;
constexpr int kSortPasses = 8;  // 8 x 8 bits >= 63-bit keys

// Device status bits (reported at the next synchronising call).
enum DevStatus : int { ST_BOX = 1, ST_CAPACITY = 2, ST_SINGULAR = 4, ST_STIR_NOISE = 8, ST_DECOMP = 16 };

// Small block of device scalars: reductions, the integrator clock and status.
struct DevScalars {
  unsigned long long box_min_ord[3];  // order-preserving encodings (open axes)
  unsigned long long box_max_ord[3];
  double box_min[3], box_max[3];      // the box used by this step
  unsigned long long hmax_ord;        // max h (cell level)
  unsigned long long minhc_ord;       // min h/c (time step)
  int cell_level;         // fine level of the cell table (= coarse + 1)
  int status;
  int max_nc, min_nc;
  unsigned long long total_nc;
  unsigned long long cand_total;  // neighbour-search candidates streamed (diagnostic)
  unsigned long long pass_total;  // warp passes of the neighbour search (diagnostic)
  double t, dt, dt_prev;
  int first;
  int pad;
  unsigned long long nbr_next;    // neighbour search: next 32-target tile (dynamic schedule)
  unsigned long long stir_step;   // STIR phases run since sph_stir_init
  unsigned long long grav_mp, grav_pp, grav_pops;  // gravity walk diagnostics (per warp sums)
  unsigned long long grav_next;   // gravity walk: next 32-target tile (dynamic schedule)
  // SFC decomposition (k_decomp.cu): the caller's all-reduced box / h_max
  // (sph_set_key_box), the reduction scratch and the split bins
  double key_box[7];              // -min x, -min y, -min z, max x, max y, max z, max h
  unsigned long long red_ord[7];
  int32_t splits[65];
  unsigned long long sort_maxrun;  // longest run of the sort's fixup (k_sort.cu)
};

// Self-gravity (k_gravity.cu).
struct GravParams {
  double G, eps, theta;
  int level;
  int fp32;  // theta > 0 and !cfg.grav_fp64: fp32 terms, fp64 accumulation
};

// Turbulence driving (k_stir.cu): the OU state and its inputs, in the arena.
constexpr int kStirModes = 61;
struct Stir {
  double* A;        // [61][6] OU state
  double* B;        // [61][6] 2 w_m A^_m (projected, weighted) of the current step
  double* w;        // [61] mode weights
  double* noise;    // [nsteps][61][6] Gaussian draws (caller's)
  int64_t nsteps;
  double sigma, t_decay, zeta;
};

// Packed fp32x2 arithmetic (FADD2/FMUL2/FFMA2 on sm_100a): two values per
// instruction (the neighbour test's candidates, gravity's fp32 terms).  Each
// half is IEEE round-to-nearest.
__device__ __forceinline__ unsigned long long pack2(float lo, float hi) {
  return ((unsigned long long)__float_as_uint(hi) << 32) | (unsigned long long)__float_as_uint(lo);
}
__device__ __forceinline__ void unpack2(unsigned long long v, float& lo, float& hi) {
  lo = __uint_as_float((uint32_t)v);
  hi = __uint_as_float((uint32_t)(v >> 32));
}
__device__ __forceinline__ unsigned long long sub2(unsigned long long a, unsigned long long b) {
  unsigned long long d;
  asm("sub.rn.f32x2 %0, %1, %2;" : "=l"(d) : "l"(a), "l"(b));
  return d;
}
__device__ __forceinline__ unsigned long long mul2(unsigned long long a, unsigned long long b) {
  unsigned long long d;
  asm("mul.rn.f32x2 %0, %1, %2;" : "=l"(d) : "l"(a), "l"(b));
  return d;
}
__device__ __forceinline__ unsigned long long fma2(unsigned long long a, unsigned long long b,
                                                   unsigned long long c) {
  unsigned long long d;
  asm("fma.rn.f32x2 %0, %1, %2, %3;" : "=l"(d) : "l"(a), "l"(b), "l"(c));
  return d;
}
__device__ __forceinline__ unsigned long long add2(unsigned long long a, unsigned long long b) {
  unsigned long long d;
  asm("add.rn.f32x2 %0, %1, %2;" : "=l"(d) : "l"(a), "l"(b));
  return d;
}
__device__ __forceinline__ unsigned long long splat2(float v) { return pack2(v, v); }

// 32-byte record: one 256-bit load (LDG.E.256 on sm_100a).
struct __align__(32) Rec4 {
  double a, b, c, d;
};
__device__ __forceinline__ Rec4 ldg4(const Rec4* p) {
  Rec4 r;
  asm("ld.global.nc.v4.f64 {%0,%1,%2,%3}, [%4];"
      : "=d"(r.a), "=d"(r.b), "=d"(r.c), "=d"(r.d)
      : "l"(p));
  return r;
}
__device__ __forceinline__ void st4(Rec4* p, double a, double b, double c, double d) {
  asm volatile("st.global.v4.f64 [%0], {%1,%2,%3,%4};" ::"l"(p), "d"(a), "d"(b), "d"(c), "d"(d)
               : "memory");
}

// Gather-friendly j-side records.  The neighbour sums
// read, per pair, whole records instead of one 8-byte word from each of up to 19
// separate arrays: 1 sector (density, IAD) or 4-5 sectors (momentum) per pair.
//   rec_d[j]       = {x, y, z, m}                                (density)
//   rec_i[j]       = {x, y, z, V = m/rho}                        (IAD)
//   rec_m[5j + 0]  = {x, y, z, wq}      wq = (pi/2h)^2            (momentum)
//   rec_m[5j + 1]  = {C11, C12, C13, wk}  wk = K/h^3
//   rec_m[5j + 2]  = {C22, C23, C33, m}
//   rec_m[5j + 3]  = {vx, vy, vz, p/rho^2}
//   rec_m[5j + 4]  = {h, c, rho, 0}      (read only for approaching pairs)
// (A chunk-major layout rec_m[k cap + j] was measured: no gain, +14 registers.)
constexpr int kRecM = 5;

// Everything the kernels need, passed by value.
struct Fields {
  int64_t n, cap;
  double* f[kNumStateF];  // current buffer
  int64_t* id;
  uint64_t* key;          // sorted keys (valid after the sort)
  double *rho, *p, *c, *vol, *prho2;
  double *wq, *wk;        // per-particle kernel factors (pi/2h)^2 and K/h^3
  double* C[6];           // 11 12 13 22 23 33
  double *ax, *ay, *az, *du;
  double *divv, *curl[3], *bal;  // IADVelocityDivCurl extras (cfg.divcurl / av_switch)
  Rec4* rec_iv;           // {vx, vy, vz, 0} gather record of the div/curl sums (EOS)
  double* phi;            // gravitational potential (GRAVITY)
  double *omega, *vsig;   // grad-h factor (GRADH), signal velocity (cfg.dt_vsig)
  uint32_t* gcell_start;  // gravity octree: leaf ranges at level grav_level
  Rec4* gmom;             // gravity octree moments, 3 records per cell, levels 0..Lt
  int32_t* nc;
  uint8_t* bnd;           // 1: the target has a ghost among its neighbours (search; multi-rank overlap)
  int32_t* nbr;           // [ngmax][cap] column-major: neighbour k of target i at nbr[k * cap + i]
  int32_t* nrows;         // neighbour-search scratch: row-major rows of the resident warps
  int64_t nrows_ld;       // their row stride (ngmax + 1 rounded up to 8: 32-B aligned rows, a spare word)
  int32_t ngmax;
  uint32_t* cell_start;   // [8^L + 1], L = fine cell level
  float4* pos4;           // fp32 (x, y, z) - box_min: neighbour-search prefilter
  Rec4* rec_d;
  Rec4* rec_i;
  Rec4* rec_m;            // [kRecM * cap]
  DevScalars* ds;
};

struct Params {
  double box_min[3], box_max[3];
  int periodic[3];
  int eos;
  double gamma, cs0, K, ng0, h_cap, k_cour, dt_max_growth;
  double av_alpha, av_beta, av_eps;
  int max_cell_level;
  int divcurl, av_switch;
  int gradh, dt_vsig, ve;
  int key_box_set;  // open axes take DevScalars::key_box (multi-rank: the global box)
  int part;         // SPH_PART_*: which targets IAD / MOMENTUM_ENERGY / EOS process (sph_set_part)
  int nbr_merge_runs;  // search: merge each cell's runs above this many runs (-1: the table size;
                       // test hook SPH_NBR_MERGE_RUNS, read at sph_init)
};

// Process-wide count of libsph kernel launches (sph_kernel_launches).
extern std::atomic<long long> g_launches;
inline void note_launch(int k = 1) { g_launches.fetch_add(k, std::memory_order_relaxed); }

// ---------------------------------------------------------------- helpers
__host__ __device__ inline int64_t div_up(int64_t a, int64_t b) { return (a + b - 1) / b; }

__device__ __forceinline__ unsigned long long ord_of(double v) {
  unsigned long long b = (unsigned long long)__double_as_longlong(v);
  return (b >> 63) ? ~b : (b | 0x8000000000000000ull);
}
__device__ __forceinline__ double unord(unsigned long long o) {
  unsigned long long b = (o >> 63) ? (o & 0x7fffffffffffffffull) : ~o;
  return __longlong_as_double((long long)b);
}

// Eight consecutive 32-bit words in one 256-bit load (coherent: the data may
// have been written earlier in the same kernel, ordered by __syncwarp).
__device__ __forceinline__ void ld8i(const int32_t* p, int (&v)[8]) {
  asm volatile("ld.global.v8.b32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
               : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7])
               : "l"(p)
               : "memory");
}

// 21-bit Morton spread / compact (x most significant in each triplet).
__device__ __forceinline__ uint64_t spread3(uint64_t v) {
  v &= 0x1fffffull;
  v = (v | v << 32) & 0x1f00000000ffffull;
  v = (v | v << 16) & 0x1f0000ff0000ffull;
  v = (v | v << 8) & 0x100f00f00f00f00full;
  v = (v | v << 4) & 0x10c30c30c30c30c3ull;
  v = (v | v << 2) & 0x1249249249249249ull;
  return v;
}
__device__ __forceinline__ uint32_t compact3(uint64_t v) {
  v &= 0x1249249249249249ull;
  v = (v ^ (v >> 2)) & 0x10c30c30c30c30c3ull;
  v = (v ^ (v >> 4)) & 0x100f00f00f00f00full;
  v = (v ^ (v >> 8)) & 0x1f0000ff0000ffull;
  v = (v ^ (v >> 16)) & 0x1f00000000ffffull;
  v = (v ^ (v >> 32)) & 0x1fffffull;
  return (uint32_t)v;
}
__device__ __forceinline__ uint64_t morton3(uint32_t ix, uint32_t iy, uint32_t iz) {
  return (spread3(ix) << 2) | (spread3(iy) << 1) | spread3(iz);
}

// Minimum image of one raw difference, exactly as the reading of item 4:
// raw difference first, then one conditional +-L (no FMA anywhere).
__device__ __forceinline__ double min_image(double dx, double L, double halfL, bool periodic) {
  if (periodic) {
    if (dx > halfL) dx = __dsub_rn(dx, L);
    else if (dx < -halfL) dx = __dadd_rn(dx, L);
  }
  return dx;
}

// sinc(x) for x^2 = t in [0, pi^2]: degree-10 polynomial in t (10 Horner FMAs),
// interpolating sin(sqrt t)/sqrt t at the 11 Chebyshev nodes of [0, pi^2]
// (coefficients from tools/sinc_fit.py, 40-digit mpmath).  Max abs error
// 2.6e-16 on [0, pi] in fp64 -- the same as the 14-term Taylor series (2.9e-16,
// SURVEY 8(d)) with 3 fewer FMAs; no sqrt/sin per pair.
__device__ __forceinline__ double sinc_t(double t) {
  double s = 1.757765687553025e-20;
  s = fma(s, t, -8.174661446309616e-18);
  s = fma(s, t, 2.810853428685386e-15);
  s = fma(s, t, -7.647114315511918e-13);
  s = fma(s, t, 1.6059041234417302e-10);
  s = fma(s, t, -2.5052108297340973e-08);
  s = fma(s, t, 2.7557319222125406e-06);
  s = fma(s, t, -0.00019841269841246913);
  s = fma(s, t, 0.008333333333333188);
  s = fma(s, t, -0.16666666666666663);
  s = fma(s, t, 1.0);
  return s;
}

// cos(x) for x^2 = t in [0, pi^2]: degree-11 polynomial in t interpolating
// cos(sqrt t) at the 12 Chebyshev nodes (tools/sinc_fit.py); max abs error
// 7.8e-16.  Used by the grad-h kernel derivative.
__device__ __forceinline__ double cos_t(double t) {
  double s = -7.989706279341135e-22;
  s = fma(s, t, 4.087216582195389e-19);
  s = fma(s, t, -1.561579798047433e-16);
  s = fma(s, t, 4.779445319504966e-14);
  s = fma(s, t, -1.1470743608679213e-11);
  s = fma(s, t, 2.0876756905345936e-09);
  s = fma(s, t, -2.7557319221730827e-07);
  s = fma(s, t, 2.4801587301548223e-05);
  s = fma(s, t, -0.0013888888888888488);
  s = fma(s, t, 0.041666666666666644);
  s = fma(s, t, -0.5);
  s = fma(s, t, 1.0);
  return s;
}

// S^6 for the kernel: W = (K/h^3) * S(pi r / 2h)^6, t = r^2 * (pi/2h)^2.
__device__ __forceinline__ double sinc6_t(double t) {
  double s = sinc_t(t);
  double s2 = s * s;
  return s2 * s2 * s2;
}

// The same polynomial with its coefficients in the constant bank (DFMA c[][]
// operands).  Used by momentum-energy, where the literal form made the compiler
// re-materialise every 64-bit coefficient with two UMOVs per use inside the
// loop (~18% of its issued instructions; 10.98 -> 10.80 ms).  Density and IAD
// keep the literal form (there the constant-bank form measured slower).
__constant__ double c_sinc_poly[11] = {
    1.757765687553025e-20,  -8.174661446309616e-18, 2.810853428685386e-15,
    -7.647114315511918e-13, 1.6059041234417302e-10, -2.5052108297340973e-08,
    2.7557319222125406e-06, -0.00019841269841246913, 0.008333333333333188,
    -0.16666666666666663,   1.0};

__device__ __forceinline__ double sinc6_t_cb(double t) {
  double s = c_sinc_poly[0];
#pragma unroll
  for (int k = 1; k < 11; ++k) s = fma(s, t, c_sinc_poly[k]);
  double s2 = s * s;
  return s2 * s2 * s2;
}

}  // namespace sph

// ---------------------------------------------------------------- launchers
// (defined in the k_*.cu files; all enqueue on `st`)
namespace sph {
void launch_reset_scalars(DevScalars* ds, const Params& P, cudaStream_t st);
void launch_box_keys(const Fields& F, const Params& P, cudaStream_t st);
void sort_workspace(int64_t cap, size_t* hist_bytes, size_t* status_bytes);
cudaError_t launch_sort(const Fields& F, uint64_t* key_in, uint64_t* key_tmp, uint32_t* val_a,
                        uint32_t* val_b, uint32_t* hist, uint32_t* status, size_t status_bytes,
                        uint32_t** perm_out, uint64_t** key_out, cudaStream_t st, int skip = 0);
void launch_permute(const Fields& Fdst, const uint32_t* perm, double* const* src,
                    const int64_t* id_src, cudaStream_t st);
void launch_cells(const Fields& F, const Params& P, int level_cap, cudaStream_t st);
void launch_neighbors(const Fields& F, const Params& P, cudaStream_t st);
constexpr int kNbrSlots = 1024;    // neighbour-search CTAs in flight (>= SMs x resident CTAs)
constexpr int kNbrSlotRows = 128;  // scratch rows per CTA (its threads)
void launch_density(const Fields& F, const Params& P, cudaStream_t st);
void launch_eos(const Fields& F, const Params& P, cudaStream_t st, bool apply_omega = false);
void launch_iad(const Fields& F, const Params& P, cudaStream_t st);
void launch_gradh(const Fields& F, const Params& P, cudaStream_t st);
// decomposition plumbing (k_decomp.cu)
constexpr int kRowDoubles = 11;     // SPH_ROW_DOUBLES
constexpr int kMaxGhostRanks = 64;
cudaError_t launch_compact(int64_t n, const uint8_t* keep, int drop, double* const* src, const int64_t* id_src,
                           double* const* dst, int64_t* id_dst, int64_t* scratch, int64_t* total,
                           cudaStream_t st, const uint64_t* drop_mask = nullptr);
cudaError_t launch_decomp_reduce(int64_t n, double* const* f, const int64_t* id, unsigned long long* ord7,
                                 double* red, cudaStream_t st);
cudaError_t launch_key_histogram(int64_t n, const uint64_t* key, const int64_t* id, int bits, int64_t* hist,
                                 cudaStream_t st);
cudaError_t launch_decomp_owners(int64_t n, const uint64_t* key, const int64_t* id, const int64_t* hist, int bits,
                                 int rank, int world, int32_t* splits, uint64_t* mig_mask, int64_t* counts,
                                 cudaStream_t st);
cudaError_t launch_decomp_ghosts(int64_t n, const uint64_t* key, int bits, int rank, int world,
                                 const int32_t* splits, const DevScalars* ds, const Params& P, uint64_t* mask,
                                 int64_t* counts, cudaStream_t st);
cudaError_t launch_route_pack(int64_t n, const uint64_t* mask, int world, double* const* src, const int64_t* id,
                              uint64_t or_id, double* rows, int64_t* pos, int64_t* scratch, int64_t* total,
                              cudaStream_t st);
cudaError_t launch_inverse_perm(int64_t n, const uint32_t* perm, uint32_t* inv, cudaStream_t st);
cudaError_t launch_map_positions(int64_t m, const int64_t* pre, int64_t first, const uint32_t* inv, int64_t* post,
                                 cudaStream_t st);
cudaError_t launch_halo(int64_t m, const int64_t* idx, double* const* f, int nf, double* buf, bool gather,
                        cudaStream_t st);
cudaError_t launch_pack_rows(int64_t m, const int64_t* idx, double* const* src, const int64_t* id,
                             uint64_t or_id, double* dst, cudaStream_t st);
cudaError_t launch_append_rows(int64_t m, int64_t n0, const double* rows, double* const* dst, int64_t* id,
                               cudaStream_t st);
cudaError_t launch_select_ghosts(int64_t n, double* const* f, const double* boxes, int R, int self,
                                 double radius, const double L[3], const int per[3], uint64_t* mask,
                                 cudaStream_t st);
cudaError_t launch_gather_field(int64_t m, const int64_t* idx, const double* f, double* dst, cudaStream_t st);
cudaError_t launch_scatter_field(int64_t m, const int64_t* idx, const double* src, double* f, cudaStream_t st);
void launch_prho2(const Fields& F, cudaStream_t st);
void launch_momentum_energy(const Fields& F, const Params& P, cudaStream_t st);
void launch_timestep(const Fields& F, const Params& P, cudaStream_t st);
void launch_update(const Fields& F, const Params& P, cudaStream_t st);
void launch_advance_time(const Fields& F, cudaStream_t st);
void launch_refresh_rec_m(const Fields& F, cudaStream_t st);
void stir_upload_modes();
void launch_stir(const Fields& F, const Params& P, const Stir& S, cudaStream_t st);
void launch_gravity(const Fields& F, const GravParams& G, cudaStream_t st);
int stir_modes(int32_t* n3);  // host: the fixed mode set (returns kStirModes)
}  // namespace sph
