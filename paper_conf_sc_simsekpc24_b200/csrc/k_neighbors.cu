// k_neighbors.cu -- phases CELLS and NEIGHBORS (items 3-4 of DESIGN.md section 3).
//
// CELLS: a uniform grid over the box at level L (2^L cells per axis) whose cells
// are exactly the level-L octree nodes of the Morton curve, so every cell is one
// contiguous range of the sorted particles: cell_start[c] .. cell_start[c+1] with
// c = key >> 3(21-L).  L is the finest level <= cap whose cell side is >= 2 h_max
// on every axis (decided on the device from the exact h_max of phase KEYS, so no
// host round trip).  HBM-bound: 8 B/particle read (key) + 4 B/cell written.
//
// NEIGHBORS: one thread per target i.  The 27 stencil cells around i's cell
// (periodic wrap or clipped at open faces, duplicates removed when 2^L < 3) are
// sorted by Morton index with a register bitonic network, so candidates are
// visited -- and neighbours appended -- in ascending particle index, the
// oracle's order.  The predicate is the oracle's exactly: raw difference,
// conditional +-L, d2 = (dx*dx + dy*dy) + dz*dz with every operation rounded
// (__dmul_rn/__dadd_rn: no FMA contraction), d2 < (2h_i)(2h_i).  Consecutive
// targets sit in the same few cells, so a warp's candidate loads are mostly
// broadcasts from L1.  Lists are stored column-major nbr[k*cap + i].
// Bound: FP64 pipe (the exact predicate costs ~15 DP ops per candidate; ~27 x
// 30 candidates per target).  Algorithmic bytes: x, y, z, h in (32 B), nc out
// (4 B) and the list out (4 B per neighbour).
#include <algorithm>

#include "sph_internal.cuh"

namespace sph {

__global__ void cell_level_kernel(DevScalars* ds, int level_cap) {
  double hmax = unord(ds->hmax_ord);
  int L = level_cap;
  while (L > 0) {
    bool ok = true;
    for (int a = 0; a < 3; ++a) {
      double side = (ds->box_max[a] - ds->box_min[a]) / (double)(1 << L);
      if (!(side >= 2.0 * hmax * (1.0 + 1e-9))) ok = false;
    }
    if (ok) break;
    --L;
  }
  ds->cell_level = L;
}

__global__ void __launch_bounds__(256) cells_kernel(int64_t n, const uint64_t* __restrict__ key,
                                                    const DevScalars* __restrict__ ds,
                                                    uint32_t* __restrict__ cell_start) {
  int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (i >= n) return;
  const int L = ds->cell_level;
  const int shift = 3 * (21 - L);
  const int64_t ncell = 1ll << (3 * L);
  int64_t ck = (int64_t)(key[i] >> shift);
  int64_t prev = i > 0 ? (int64_t)(key[i - 1] >> shift) : -1;
  for (int64_t c = prev + 1; c <= ck; ++c) cell_start[c] = (uint32_t)i;
  if (i == n - 1)
    for (int64_t c = ck + 1; c <= ncell; ++c) cell_start[c] = (uint32_t)n;
}

void launch_cells(const Fields& F, const Params& P, int level_cap, cudaStream_t st) {
  (void)P;
  cell_level_kernel<<<1, 1, 0, st>>>(F.ds, level_cap); note_launch();
  if (F.n > 0) {
    cells_kernel<<<(unsigned)div_up(F.n, 256), 256, 0, st>>>(F.n, F.key, F.ds, F.cell_start);
    note_launch();
  }
}

template <int N>
__device__ __forceinline__ void bitonic_sort(uint32_t (&a)[N]) {
#pragma unroll
  for (int k = 2; k <= N; k <<= 1)
#pragma unroll
    for (int j = k >> 1; j > 0; j >>= 1)
#pragma unroll
      for (int i = 0; i < N; ++i) {
        const int l = i ^ j;
        if (l > i) {
          uint32_t x = a[i], y = a[l];
          uint32_t lo = min(x, y), hi = max(x, y);
          if ((i & k) == 0) {
            a[i] = lo;
            a[l] = hi;
          } else {
            a[i] = hi;
            a[l] = lo;
          }
        }
      }
}

constexpr int kNbrThreads = 128;
constexpr uint32_t kNoCell = 0xffffffffu;

__global__ void __launch_bounds__(kNbrThreads) neighbors_kernel(Fields F, Params P) {
  __shared__ uint32_t s_cells[27][kNbrThreads];
  const int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  const bool active = i < F.n;
  int cnt = 0;
  if (active) {
    const DevScalars* ds = F.ds;
    const int L = ds->cell_level;
    const int nside = 1 << L;
    const uint64_t key = F.key[i];
    const int cx = (int)(compact3(key >> 2) >> (21 - L));
    const int cy = (int)(compact3(key >> 1) >> (21 - L));
    const int cz = (int)(compact3(key) >> (21 - L));
    uint32_t ck[32];
#pragma unroll
    for (int s = 0; s < 32; ++s) {
      if (s >= 27) {
        ck[s] = kNoCell;
        continue;
      }
      int o[3] = {s / 9 - 1, (s / 3) % 3 - 1, s % 3 - 1};
      int c[3] = {cx + o[0], cy + o[1], cz + o[2]};
      bool ok = true;
#pragma unroll
      for (int a = 0; a < 3; ++a) {
        if (c[a] < 0 || c[a] >= nside) {
          if (P.periodic[a]) c[a] = (c[a] + nside) % nside;
          else ok = false;
        }
      }
      ck[s] = ok ? (uint32_t)morton3((uint32_t)c[0], (uint32_t)c[1], (uint32_t)c[2]) : kNoCell;
    }
    bitonic_sort<32>(ck);
#pragma unroll
    for (int s = 0; s < 27; ++s) s_cells[s][threadIdx.x] = ck[s];

    const double xi = F.f[FX][i], yi = F.f[FY][i], zi = F.f[FZ][i], hi = F.f[FH][i];
    const double r2max = (2.0 * hi) * (2.0 * hi);
    double L0 = ds->box_max[0] - ds->box_min[0], L1 = ds->box_max[1] - ds->box_min[1],
           L2 = ds->box_max[2] - ds->box_min[2];
    double H0 = 0.5 * L0, H1 = 0.5 * L1, H2 = 0.5 * L2;
    const bool p0 = P.periodic[0], p1 = P.periodic[1], p2 = P.periodic[2];
    const double* __restrict__ X = F.f[FX];
    const double* __restrict__ Y = F.f[FY];
    const double* __restrict__ Z = F.f[FZ];
    int32_t* __restrict__ nbr = F.nbr;
    const int64_t cap = F.cap;
    const int ngmax = F.ngmax;
    uint32_t prev = kNoCell;
    for (int s = 0; s < 27; ++s) {
      const uint32_t cell = s_cells[s][threadIdx.x];
      if (cell == kNoCell) break;
      if (cell == prev) continue;
      prev = cell;
      const uint32_t j0 = F.cell_start[cell], j1 = F.cell_start[cell + 1];
      for (uint32_t j = j0; j < j1; ++j) {
        if ((int64_t)j == i) continue;
        double dx = min_image(__dsub_rn(xi, __ldg(X + j)), L0, H0, p0);
        double dy = min_image(__dsub_rn(yi, __ldg(Y + j)), L1, H1, p1);
        double dz = min_image(__dsub_rn(zi, __ldg(Z + j)), L2, H2, p2);
        double d2 = __dadd_rn(__dadd_rn(__dmul_rn(dx, dx), __dmul_rn(dy, dy)), __dmul_rn(dz, dz));
        if (d2 < r2max) {
          if (cnt < ngmax) nbr[(int64_t)cnt * cap + i] = (int32_t)j;
          ++cnt;
        }
      }
    }
    F.nc[i] = cnt;
  }
  // nc statistics (min, max, total) and the capacity flag.
  int mn = active ? cnt : 0x7fffffff, mx = active ? cnt : 0;
  unsigned long long tot = active ? (unsigned long long)cnt : 0ull;
#pragma unroll
  for (int off = 16; off > 0; off >>= 1) {
    mn = min(mn, __shfl_xor_sync(0xffffffffu, mn, off));
    mx = max(mx, __shfl_xor_sync(0xffffffffu, mx, off));
    tot += __shfl_xor_sync(0xffffffffu, tot, off);
  }
  if ((threadIdx.x & 31) == 0 && mn != 0x7fffffff) {  // warp had an active lane
    atomicMin(&F.ds->min_nc, mn);
    atomicMax(&F.ds->max_nc, mx);
    atomicAdd(&F.ds->total_nc, tot);
    if (mx > F.ngmax) atomicOr(&F.ds->status, (int)ST_CAPACITY);
  }
}

void launch_neighbors(const Fields& F, const Params& P, cudaStream_t st) {
  if (F.n == 0) return;
  neighbors_kernel<<<(unsigned)div_up(F.n, kNbrThreads), kNbrThreads, 0, st>>>(F, P); note_launch();
}

}  // namespace sph
