// k_keys.cu -- phase KEYS: box reduction and 63-bit Morton keys (item 1-2 of
// DESIGN.md section 3; DomainDecompAndSync's "particle keys").
//
// Roofline: HBM-bound.  Algorithmic bytes per particle: read x, y, z (24 B, twice
// when an axis is open: once for the box), read h (8 B, for h_max), write the key
// (8 B).  The box min/max and h_max are exact (order-preserving integer atomics),
// so keys are bit-identical to the oracle's.
#include "sph_internal.cuh"

namespace sph {

__global__ void reset_scalars_kernel(DevScalars* ds) {
  for (int a = 0; a < 3; ++a) {
    ds->box_min_ord[a] = ~0ull;
    ds->box_max_ord[a] = 0ull;
  }
  ds->hmax_ord = 0ull;
  ds->minhc_ord = ~0ull;
  ds->sort_maxrun = 0ull;
  ds->status = 0;
  ds->max_nc = 0;
  ds->min_nc = 0x7fffffff;
  ds->total_nc = 0ull;
}

void launch_reset_scalars(DevScalars* ds, const Params&, cudaStream_t st) {
  reset_scalars_kernel<<<1, 1, 0, st>>>(ds); note_launch();
}

constexpr int kBoxThreads = 256;

// Min/max of x, y, z over all particles (open axes) and max h.
__global__ void __launch_bounds__(kBoxThreads) box_reduce_kernel(int64_t n, const double* __restrict__ x,
                                                  const double* __restrict__ y,
                                                  const double* __restrict__ z,
                                                  const double* __restrict__ h, DevScalars* ds,
                                                  int need_box) {
  unsigned long long mn[3] = {~0ull, ~0ull, ~0ull}, mx[3] = {0, 0, 0}, hm = 0;
  const double* c[3] = {x, y, z};
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n;
       i += (int64_t)gridDim.x * blockDim.x) {
    if (need_box) {
#pragma unroll
      for (int a = 0; a < 3; ++a) {
        unsigned long long o = ord_of(__ldg(c[a] + i));
        mn[a] = o < mn[a] ? o : mn[a];
        mx[a] = o > mx[a] ? o : mx[a];
      }
    }
    unsigned long long oh = ord_of(__ldg(h + i));
    hm = oh > hm ? oh : hm;
  }
#pragma unroll
  for (int off = 16; off > 0; off >>= 1) {
#pragma unroll
    for (int a = 0; a < 3; ++a) {
      unsigned long long t = __shfl_xor_sync(0xffffffffu, mn[a], off);
      mn[a] = t < mn[a] ? t : mn[a];
      t = __shfl_xor_sync(0xffffffffu, mx[a], off);
      mx[a] = t > mx[a] ? t : mx[a];
    }
    unsigned long long t = __shfl_xor_sync(0xffffffffu, hm, off);
    hm = t > hm ? t : hm;
  }
  if ((threadIdx.x & 31) == 0) {
    if (need_box) {
      for (int a = 0; a < 3; ++a) {
        atomicMin(&ds->box_min_ord[a], mn[a]);
        atomicMax(&ds->box_max_ord[a], mx[a]);
      }
    }
    atomicMax(&ds->hmax_ord, hm);
  }
}

// Resolves the step's box: periodic axes from the configuration, open axes from
// the reduction; flags a degenerate open axis.
__global__ void box_finalize_kernel(DevScalars* ds, Params P, int64_t n) {
  for (int a = 0; a < 3; ++a) {
    if (P.periodic[a]) {
      ds->box_min[a] = P.box_min[a];
      ds->box_max[a] = P.box_max[a];
    } else if (P.key_box_set) {  // the global box of a decomposed run (sph_set_key_box)
      const double lo = -ds->key_box[a], hi = ds->key_box[3 + a];
      ds->box_min[a] = lo;
      ds->box_max[a] = hi;
      if (!(hi > lo)) ds->status |= ST_BOX;
    } else {
      double lo = unord(ds->box_min_ord[a]), hi = unord(ds->box_max_ord[a]);
      ds->box_min[a] = lo;
      ds->box_max[a] = hi;
      if (n > 0 && !(hi > lo)) ds->status |= ST_BOX;
    }
  }
}

// s = (x - xmin)/L (IEEE division); ix = min(floor(s * 2^21), 2^21 - 1), >= 0.
__device__ __forceinline__ uint32_t coord21(double v, double lo, double L) {
  double s = __ddiv_rn(__dsub_rn(v, lo), L);
  double f = floor(__dmul_rn(s, 2097152.0));
  f = f < 0.0 ? 0.0 : f;
  f = f > 2097151.0 ? 2097151.0 : f;
  return (uint32_t)f;
}

__global__ void __launch_bounds__(256) keys_kernel(int64_t n, const double* __restrict__ x,
                                                  const double* __restrict__ y,
                                                  const double* __restrict__ z,
                                                  const DevScalars* __restrict__ ds,
                                                  uint64_t* __restrict__ key) {
  int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (i >= n) return;
  double lo0 = ds->box_min[0], lo1 = ds->box_min[1], lo2 = ds->box_min[2];
  double L0 = ds->box_max[0] - lo0, L1 = ds->box_max[1] - lo1, L2 = ds->box_max[2] - lo2;
  key[i] = morton3(coord21(x[i], lo0, L0), coord21(y[i], lo1, L1), coord21(z[i], lo2, L2));
}

void launch_box_keys(const Fields& F, const Params& P, cudaStream_t st) {
  int need_box = !(P.periodic[0] && P.periodic[1] && P.periodic[2]);
  if (F.n > 0) {
    int blocks = (int)std::min<int64_t>(div_up(F.n, kBoxThreads), 148 * 8);
    box_reduce_kernel<<<blocks, kBoxThreads, 0, st>>>(F.n, F.f[FX], F.f[FY], F.f[FZ], F.f[FH], F.ds,
                                                      need_box); note_launch();
  }
  box_finalize_kernel<<<1, 1, 0, st>>>(F.ds, P, F.n); note_launch();
  if (F.n > 0) {
    keys_kernel<<<(unsigned)div_up(F.n, 256), 256, 0, st>>>(F.n, F.f[FX], F.f[FY], F.f[FZ], F.ds,
                                                           F.key);
    note_launch();
  }
}

}  // namespace sph
