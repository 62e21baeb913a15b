// k_decomp.cu -- device plumbing of the decomposed step (the
// functions are declared in include/sph.h, "Device-side plumbing").  Nothing
// here computes a value of the method: the kernels select, move and pack
// particles so that decomp.py never copies the whole state through PyTorch.
// All are HBM-bound streaming passes (one read + one write of the moved fields).
#include "sph_internal.cuh"

namespace sph {

constexpr int kCompactThreads = 1024;

__device__ __forceinline__ bool keep_of(const uint8_t* keep, const int64_t* id, int64_t i, int drop) {
  return (keep == nullptr || keep[i] != 0) && !(drop && (id[i] & SPH_GHOST_BIT));
}

// 1. kept count per block
__global__ void __launch_bounds__(kCompactThreads) compact_count_kernel(int64_t n, const uint8_t* keep,
                                                                       const int64_t* id, int drop,
                                                                       int64_t* block_count) {
  const int64_t i = blockIdx.x * (int64_t)kCompactThreads + threadIdx.x;
  const int k = __syncthreads_count(i < n && keep_of(keep, id, i, drop));
  if (threadIdx.x == 0) block_count[blockIdx.x] = k;
}

// 2. exclusive scan of the block counts (one block; nb <= 2^20 / 1024 * ...)
__global__ void __launch_bounds__(1024) compact_scan_kernel(int64_t nb, int64_t* block_count,
                                                            int64_t* total) {
  __shared__ int64_t part[1024];
  const int t = threadIdx.x;
  const int64_t per = (nb + 1023) / 1024;
  const int64_t b0 = t * per, b1 = min(nb, b0 + per);
  int64_t s = 0;
  for (int64_t b = b0; b < b1; ++b) s += block_count[b];
  part[t] = s;
  __syncthreads();
  for (int off = 1; off < 1024; off <<= 1) {
    const int64_t v = t >= off ? part[t - off] : 0;
    __syncthreads();
    part[t] += v;
    __syncthreads();
  }
  int64_t run = part[t] - s;  // exclusive prefix of this thread's range
  for (int64_t b = b0; b < b1; ++b) {
    const int64_t c = block_count[b];
    block_count[b] = run;
    run += c;
  }
  if (t == 1023) *total = part[1023];
}

struct StatePtrs {
  const double* src[kNumStateF];
  double* dst[kNumStateF];
};

// 3. scatter of the kept particles, order preserved (block-local ranks by
// warp ballots)
__global__ void __launch_bounds__(kCompactThreads) compact_scatter_kernel(int64_t n, const uint8_t* keep,
                                                                         const int64_t* id_src, int drop,
                                                                         const int64_t* block_off,
                                                                         StatePtrs S, int64_t* id_dst) {
  __shared__ int warp_off[kCompactThreads / 32];
  const int64_t i = blockIdx.x * (int64_t)kCompactThreads + threadIdx.x;
  const bool k = i < n && keep_of(keep, id_src, i, drop);
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const uint32_t b = __ballot_sync(0xffffffffu, k);
  if (lane == 0) warp_off[warp] = __popc(b);
  __syncthreads();
  if (threadIdx.x == 0) {
    int run = 0;
    for (int w = 0; w < kCompactThreads / 32; ++w) {
      const int c = warp_off[w];
      warp_off[w] = run;
      run += c;
    }
  }
  __syncthreads();
  if (!k) return;
  const int64_t o = block_off[blockIdx.x] + warp_off[warp] + __popc(b & ((1u << lane) - 1u));
#pragma unroll
  for (int f = 0; f < kNumStateF; ++f) S.dst[f][o] = S.src[f][i];
  id_dst[o] = id_src[i];
}

cudaError_t launch_compact(int64_t n, const uint8_t* keep, int drop, double* const* src, const int64_t* id_src,
                           double* const* dst, int64_t* id_dst, int64_t* scratch, int64_t* total,
                           cudaStream_t st) {
  const int64_t nb = div_up(n, kCompactThreads);
  if (n == 0) return cudaMemsetAsync(total, 0, sizeof(int64_t), st);
  compact_count_kernel<<<(unsigned)nb, kCompactThreads, 0, st>>>(n, keep, id_src, drop, scratch);
  compact_scan_kernel<<<1, 1024, 0, st>>>(nb, scratch, total);
  StatePtrs S;
  for (int f = 0; f < kNumStateF; ++f) {
    S.src[f] = src[f];
    S.dst[f] = dst[f];
  }
  compact_scatter_kernel<<<(unsigned)nb, kCompactThreads, 0, st>>>(n, keep, id_src, drop, scratch, S, id_dst);
  note_launch(3);
  return cudaGetLastError();
}

__global__ void __launch_bounds__(256) pack_rows_kernel(int64_t m, const int64_t* __restrict__ idx, StatePtrs S,
                                                        const int64_t* __restrict__ id, uint64_t or_id,
                                                        double* __restrict__ dst) {
  const int64_t r = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (r >= m) return;
  const int64_t i = idx[r];
  double* row = dst + r * kRowDoubles;
#pragma unroll
  for (int f = 0; f < kNumStateF; ++f) row[f] = S.src[f][i];
  row[kNumStateF] = __longlong_as_double((long long)((uint64_t)id[i] | or_id));
}

cudaError_t launch_pack_rows(int64_t m, const int64_t* idx, double* const* src, const int64_t* id,
                             uint64_t or_id, double* dst, cudaStream_t st) {
  if (m == 0) return cudaSuccess;
  StatePtrs S;
  for (int f = 0; f < kNumStateF; ++f) {
    S.src[f] = src[f];
    S.dst[f] = nullptr;
  }
  pack_rows_kernel<<<(unsigned)div_up(m, 256), 256, 0, st>>>(m, idx, S, id, or_id, dst);
  note_launch();
  return cudaGetLastError();
}

__global__ void __launch_bounds__(256) append_rows_kernel(int64_t m, int64_t n0, const double* __restrict__ rows,
                                                          StatePtrs S, int64_t* __restrict__ id) {
  const int64_t r = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (r >= m) return;
  const double* row = rows + r * kRowDoubles;
#pragma unroll
  for (int f = 0; f < kNumStateF; ++f) S.dst[f][n0 + r] = row[f];
  id[n0 + r] = (int64_t)__double_as_longlong(row[kNumStateF]);
}

cudaError_t launch_append_rows(int64_t m, int64_t n0, const double* rows, double* const* dst, int64_t* id,
                               cudaStream_t st) {
  if (m == 0) return cudaSuccess;
  StatePtrs S;
  for (int f = 0; f < kNumStateF; ++f) {
    S.src[f] = nullptr;
    S.dst[f] = dst[f];
  }
  append_rows_kernel<<<(unsigned)div_up(m, 256), 256, 0, st>>>(m, n0, rows, S, id);
  note_launch();
  return cudaGetLastError();
}

struct GhostBoxes {
  double b[kMaxGhostRanks][6];
  double L[3];
  int per[3];
  int R, self;
  double radius;
};

// minimum-image distance of (x, y, z) to each box (the same arithmetic as
// decomp.box_distance: per axis the smallest clamp(max(lo - x', x' - hi), 0)
// over the images x' = x + k L, k in {-1, 0, 1} on periodic axes)
__global__ void __launch_bounds__(256) select_ghosts_kernel(int64_t n, const double* __restrict__ x,
                                                            const double* __restrict__ y,
                                                            const double* __restrict__ z, GhostBoxes G,
                                                            uint64_t* __restrict__ mask) {
  const int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (i >= n) return;
  const double p[3] = {x[i], y[i], z[i]};
  uint64_t m = 0;
  for (int r = 0; r < G.R; ++r) {
    if (r == G.self || !(G.b[r][0] <= G.b[r][3])) continue;
    double d2 = 0.0;
#pragma unroll
    for (int a = 0; a < 3; ++a) {
      const double lo = G.b[r][a], hi = G.b[r][3 + a];
      double best = fmax(fmax(lo - p[a], p[a] - hi), 0.0);
      if (G.per[a]) {
        for (int k = -1; k <= 1; k += 2) {
          const double xa = p[a] + k * G.L[a];
          best = fmin(best, fmax(fmax(lo - xa, xa - hi), 0.0));
        }
      }
      d2 += best * best;
    }
    if (sqrt(d2) < G.radius) m |= 1ull << r;
  }
  mask[i] = m;
}

cudaError_t launch_select_ghosts(int64_t n, double* const* f, const double* boxes, int R, int self,
                                 double radius, const double L[3], const int per[3], uint64_t* mask,
                                 cudaStream_t st) {
  if (n == 0) return cudaSuccess;
  GhostBoxes G;
  for (int r = 0; r < R; ++r)
    for (int k = 0; k < 6; ++k) G.b[r][k] = boxes[6 * r + k];
  for (int a = 0; a < 3; ++a) {
    G.L[a] = L[a];
    G.per[a] = per[a];
  }
  G.R = R;
  G.self = self;
  G.radius = radius;
  select_ghosts_kernel<<<(unsigned)div_up(n, 256), 256, 0, st>>>(n, f[FX], f[FY], f[FZ], G, mask);
  note_launch();
  return cudaGetLastError();
}

__global__ void __launch_bounds__(256) gather_kernel(int64_t m, const int64_t* __restrict__ idx,
                                                     const double* __restrict__ f, double* __restrict__ dst) {
  const int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (k < m) dst[k] = f[idx[k]];
}

__global__ void __launch_bounds__(256) scatter_kernel(int64_t m, const int64_t* __restrict__ idx,
                                                      const double* __restrict__ src, double* __restrict__ f) {
  const int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (k < m) f[idx[k]] = src[k];
}

cudaError_t launch_gather_field(int64_t m, const int64_t* idx, const double* f, double* dst, cudaStream_t st) {
  if (m == 0) return cudaSuccess;
  gather_kernel<<<(unsigned)div_up(m, 256), 256, 0, st>>>(m, idx, f, dst);
  note_launch();
  return cudaGetLastError();
}

cudaError_t launch_scatter_field(int64_t m, const int64_t* idx, const double* src, double* f, cudaStream_t st) {
  if (m == 0) return cudaSuccess;
  scatter_kernel<<<(unsigned)div_up(m, 256), 256, 0, st>>>(m, idx, src, f);
  note_launch();
  return cudaGetLastError();
}

}  // namespace sph
