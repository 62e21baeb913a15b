// k_decomp.cu -- device plumbing of the decomposed step (the
// functions are declared in include/sph.h, "Device-side plumbing").  Nothing
// here computes a value of the method: the kernels select, move and pack
// particles so that decomp.py never copies the whole state through PyTorch.
// All are HBM-bound streaming passes (one read + one write of the moved fields).
#include "sph_internal.cuh"

namespace sph {

constexpr int kCompactThreads = 1024;

__device__ __forceinline__ bool keep_of(const uint8_t* keep, const int64_t* id, int64_t i, int drop,
                                        const uint64_t* drop_mask = nullptr) {
  return (keep == nullptr || keep[i] != 0) && !(drop && (id[i] & SPH_GHOST_BIT)) &&
         (drop_mask == nullptr || drop_mask[i] == 0ull);
}

// 1. kept count per block
__global__ void __launch_bounds__(kCompactThreads) compact_count_kernel(int64_t n, const uint8_t* keep,
                                                                       const int64_t* id, int drop,
                                                                       const uint64_t* drop_mask,
                                                                       int64_t* block_count) {
  const int64_t i = blockIdx.x * (int64_t)kCompactThreads + threadIdx.x;
  const int k = __syncthreads_count(i < n && keep_of(keep, id, i, drop, drop_mask));
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
                                                                         const uint64_t* drop_mask,
                                                                         const int64_t* block_off,
                                                                         StatePtrs S, int64_t* id_dst) {
  __shared__ int warp_off[kCompactThreads / 32];
  const int64_t i = blockIdx.x * (int64_t)kCompactThreads + threadIdx.x;
  const bool k = i < n && keep_of(keep, id_src, i, drop, drop_mask);
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
                           cudaStream_t st, const uint64_t* drop_mask) {
  const int64_t nb = div_up(n, kCompactThreads);
  if (n == 0) return cudaMemsetAsync(total, 0, sizeof(int64_t), st);
  compact_count_kernel<<<(unsigned)nb, kCompactThreads, 0, st>>>(n, keep, id_src, drop, drop_mask, scratch);
  compact_scan_kernel<<<1, 1024, 0, st>>>(nb, scratch, total);
  StatePtrs S;
  for (int f = 0; f < kNumStateF; ++f) {
    S.src[f] = src[f];
    S.dst[f] = dst[f];
  }
  compact_scatter_kernel<<<(unsigned)nb, kCompactThreads, 0, st>>>(n, keep, id_src, drop, drop_mask, scratch, S,
                                                                   id_dst);
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

// =============================================================================
// SFC decomposition on the device: box / h_max reduction, key
// histogram, split points and owners, cell-stencil ghost routing, grouped row
// packing.  decomp.py only issues the collectives between these calls.
// =============================================================================
namespace sph {

// ---- box and h_max of the held non-ghost particles, as 7 order codes
// (max of -x, -y, -z, x, y, z, h): one MAX all-reduce over ranks gives the
// global box and h_max exactly.
__global__ void __launch_bounds__(256) decomp_reduce_kernel(int64_t n, const double* __restrict__ x,
                                                            const double* __restrict__ y,
                                                            const double* __restrict__ z,
                                                            const double* __restrict__ h,
                                                            const int64_t* __restrict__ id,
                                                            unsigned long long* ord7) {
  unsigned long long m[7];
#pragma unroll
  for (int k = 0; k < 7; ++k) m[k] = 0ull;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    if (id[i] & SPH_GHOST_BIT) continue;
    const double v[7] = {-x[i], -y[i], -z[i], x[i], y[i], z[i], h[i]};
#pragma unroll
    for (int k = 0; k < 7; ++k) {
      const unsigned long long o = ord_of(v[k]);
      m[k] = o > m[k] ? o : m[k];
    }
  }
#pragma unroll
  for (int off = 16; off > 0; off >>= 1)
#pragma unroll
    for (int k = 0; k < 7; ++k) {
      const unsigned long long t = __shfl_xor_sync(0xffffffffu, m[k], off);
      m[k] = t > m[k] ? t : m[k];
    }
  if ((threadIdx.x & 31) == 0)
#pragma unroll
    for (int k = 0; k < 7; ++k)
      if (m[k]) atomicMax(ord7 + k, m[k]);
}

__global__ void decomp_reduce_finish_kernel(unsigned long long* ord7, double* red) {
  const int k = threadIdx.x;
  if (k < 7) {
    // nothing held: -inf, neutral for the MAX all-reduce
    red[k] = ord7[k] ? unord(ord7[k]) : -INFINITY;
    ord7[k] = 0ull;  // ready for the next call
  }
}

cudaError_t launch_decomp_reduce(int64_t n, double* const* f, const int64_t* id, unsigned long long* ord7,
                                 double* red, cudaStream_t st) {
  if (n > 0) {
    const int blocks = (int)std::min<int64_t>(div_up(n, 256), 148 * 8);
    decomp_reduce_kernel<<<blocks, 256, 0, st>>>(n, f[FX], f[FY], f[FZ], f[FH], id, ord7);
    note_launch();
  }
  decomp_reduce_finish_kernel<<<1, 32, 0, st>>>(ord7, red);
  note_launch();
  return cudaGetLastError();
}

// ---- histogram of the top `bits` key bits
// (the keys are nearly sorted, so a warp's particles share one or two bins:
// one atomic per distinct bin per warp)
__global__ void __launch_bounds__(256) key_hist_kernel(int64_t n, const uint64_t* __restrict__ key,
                                                       const int64_t* __restrict__ id, int bits,
                                                       unsigned long long* hist) {
  const int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  const bool live = i < n && !(id[i] & SPH_GHOST_BIT);
  const unsigned long long b = live ? (key[i] >> (63 - bits)) : ~0ull;
  const uint32_t peers = __match_any_sync(0xffffffffu, b);
  if (live && (peers & ((1u << (threadIdx.x & 31)) - 1u)) == 0) atomicAdd(hist + b, (unsigned long long)__popc(peers));
}

cudaError_t launch_key_histogram(int64_t n, const uint64_t* key, const int64_t* id, int bits, int64_t* hist,
                                 cudaStream_t st) {
  cudaError_t e = cudaMemsetAsync(hist, 0, sizeof(int64_t) << bits, st);
  if (e != cudaSuccess || n == 0) return e;
  key_hist_kernel<<<(unsigned)div_up(n, 256), 256, 0, st>>>(n, key, id, bits, (unsigned long long*)hist);
  note_launch();
  return cudaGetLastError();
}

// ---- split points: s_0 = 0, s_world = 2^bits, and for 0 < r < world the first
// bin whose inclusive prefix count exceeds floor(total r / world) (one block)
__global__ void __launch_bounds__(1024) splits_kernel(const int64_t* __restrict__ hist, int bits, int world,
                                                      int32_t* __restrict__ splits) {
  __shared__ int64_t part[1024];
  const int t = threadIdx.x;
  const int nb = 1 << bits;
  const int per = (nb + 1023) / 1024;
  const int b0 = min(nb, t * per), b1 = min(nb, b0 + per);
  int64_t s = 0;
  for (int b = b0; b < b1; ++b) s += hist[b];
  part[t] = s;
  __syncthreads();
  for (int off = 1; off < 1024; off <<= 1) {
    const int64_t v = t >= off ? part[t - off] : 0;
    __syncthreads();
    part[t] += v;
    __syncthreads();
  }
  const int64_t total = part[1023];
  int64_t run = part[t] - s;  // exclusive prefix before b0
  for (int b = b0; b < b1; ++b) {
    const int64_t before = run;
    run += hist[b];
    // bin b is the split of every r whose target lies in [before, run)
    for (int r = 1; r < world; ++r) {
      const int64_t target = total * r / world;
      if (target >= before && target < run) splits[r] = b;
    }
  }
  if (t == 0) {
    splits[0] = 0;
    splits[world] = nb;
  }
  // targets never reached (total 0, or every count before the end): past the end
  __syncthreads();
  if (t == 0)
    for (int r = 1; r < world; ++r)
      if (total * r / world >= total) splits[r] = nb;
}

__device__ __forceinline__ int owner_of_bin(const int32_t* s, int world, int bin) {
  int lo = 0, hi = world;  // s[lo] <= bin < s[hi]
  while (hi - lo > 1) {
    const int mid = (lo + hi) >> 1;
    if (s[mid] <= bin) lo = mid;
    else hi = mid;
  }
  return lo;
}

__global__ void __launch_bounds__(256) owners_kernel(int64_t n, const uint64_t* __restrict__ key,
                                                     const int64_t* __restrict__ id, int bits,
                                                     int rank, int world, const int32_t* __restrict__ splits,
                                                     uint64_t* __restrict__ mig_mask,
                                                     unsigned long long* __restrict__ counts) {
  __shared__ int32_t s[kMaxGhostRanks + 1];
  __shared__ unsigned long long bc[kMaxGhostRanks];  // this block's count per owner
  if (threadIdx.x <= world) s[threadIdx.x] = splits[threadIdx.x];
  if (threadIdx.x < world) bc[threadIdx.x] = 0ull;
  __syncthreads();
  const int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  // last step's ghosts are neither owned nor sent (sph_decomp_drop removes them)
  const bool live = i < n && !(id[i] & SPH_GHOST_BIT);
  const int o = live ? owner_of_bin(s, world, (int)(key[i] >> (63 - bits))) : -1;
  if (i < n) mig_mask[i] = (!live || o == rank) ? 0ull : (1ull << o);
  // one shared-memory add per distinct owner per warp, one global add per
  // owner per block (an owner holds long runs of the sorted keys)
  const uint32_t peers = __match_any_sync(0xffffffffu, o);
  if (live && (peers & ((1u << (threadIdx.x & 31)) - 1u)) == 0) atomicAdd(bc + o, (unsigned long long)__popc(peers));
  __syncthreads();
  if (threadIdx.x < world && bc[threadIdx.x]) atomicAdd(counts + threadIdx.x, bc[threadIdx.x]);
}

cudaError_t launch_decomp_owners(int64_t n, const uint64_t* key, const int64_t* id, const int64_t* hist, int bits,
                                 int rank, int world, int32_t* splits, uint64_t* mig_mask, int64_t* counts,
                                 cudaStream_t st) {
  splits_kernel<<<1, 1024, 0, st>>>(hist, bits, world, splits);
  note_launch();
  cudaError_t e = cudaMemsetAsync(counts, 0, sizeof(int64_t) * world, st);
  if (e != cudaSuccess) return e;
  if (n > 0) {
    owners_kernel<<<(unsigned)div_up(n, 256), 256, 0, st>>>(n, key, id, bits, rank, world, splits, mig_mask,
                                                            (unsigned long long*)counts);
    note_launch();
  }
  return cudaGetLastError();
}

// ---- ghost routing by cells: level L = finest with box side / 2^L >= 2 h_max
// on every axis.  Particle i is sent to every rank owning a key of one of the
// 27 level-L cells around its own (periodic wrap, clipped at open faces).  A
// particle within 2 h_max of a particle j lies in a cell adjacent to j's cell,
// so j's owner receives it: the halo is conservative.
__device__ uint64_t stencil_owners(uint64_t cell, int o, int bits, int world, const int32_t* s, int L,
                                   const Params& P);

__global__ void __launch_bounds__(256) ghost_route_kernel(int64_t n, const uint64_t* __restrict__ key, int bits,
                                                          int rank, int world, const int32_t* __restrict__ splits,
                                                          const DevScalars* __restrict__ ds, Params P,
                                                          uint64_t* __restrict__ mask,
                                                          unsigned long long* __restrict__ counts) {
  __shared__ int32_t s[kMaxGhostRanks + 1];
  __shared__ int sL;
  __shared__ unsigned long long bc[kMaxGhostRanks];
  if (threadIdx.x < world) bc[threadIdx.x] = 0ull;
  if (threadIdx.x <= world) s[threadIdx.x] = splits[threadIdx.x];
  if (threadIdx.x == 0) {
    const double hmax = ds->key_box[6];
    int L = 21;
    while (L > 0) {
      bool ok = true;
      for (int a = 0; a < 3; ++a) {
        const double side = (ds->box_max[a] - ds->box_min[a]) / (double)(1 << L);
        if (!(side >= 2.0 * hmax * (1.0 + 1e-9))) ok = false;
      }
      if (ok) break;
      --L;
    }
    sL = L;
  }
  __syncthreads();
  const int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  const int lane = threadIdx.x & 31;
  const int L = sL;
  // every particle of a level-L cell has the cell's mask: the warp computes it
  // once per distinct cell (the held keys are nearly sorted: 1-2 cells per
  // warp), one stencil cell per lane, OR-reduced
  const uint64_t cell = i < n ? (key[i] >> (3 * (21 - L))) : ~0ull;
  uint32_t todo = __ballot_sync(0xffffffffu, i < n);
  uint64_t m = 0;
  while (todo) {
    const int lead = __ffs(todo) - 1;
    const uint64_t c = __shfl_sync(0xffffffffu, cell, lead);
    const uint64_t part = lane < 27 ? stencil_owners(c, lane, bits, world, s, L, P) : 0ull;
    const uint32_t lo = __reduce_or_sync(0xffffffffu, (uint32_t)part);
    const uint32_t hi = __reduce_or_sync(0xffffffffu, (uint32_t)(part >> 32));
    const uint32_t mine = __ballot_sync(0xffffffffu, cell == c);
    if (cell == c) m = (((uint64_t)hi << 32) | lo) & ~(1ull << rank);
    todo &= ~mine;
  }
  if (i < n) mask[i] = m;
  for (int r = 0; r < world; ++r) {  // one shared add per rank per warp, one global add per block
    const uint32_t b = __ballot_sync(0xffffffffu, (m >> r) & 1ull);
    if ((threadIdx.x & 31) == 0 && b) atomicAdd(bc + r, (unsigned long long)__popc(b));
  }
  __syncthreads();
  if (threadIdx.x < world && bc[threadIdx.x]) atomicAdd(counts + threadIdx.x, bc[threadIdx.x]);
}

__device__ uint64_t stencil_owners(uint64_t cell, int o, int bits, int world, const int32_t* s, int L,
                                   const Params& P) {
  // the ranks owning a key of stencil cell o (0..26) around level-L cell `cell`
  const int lb = bits / 3;  // histogram bins are the level-lb cells
  const int nside = 1 << L;
  const int c[3] = {(int)compact3(cell >> 2), (int)compact3(cell >> 1), (int)compact3(cell)};
  int u[3] = {c[0] + o / 9 - 1, c[1] + (o / 3) % 3 - 1, c[2] + o % 3 - 1};
#pragma unroll
  for (int a = 0; a < 3; ++a) {
    if (u[a] < 0 || u[a] >= nside) {
      if (P.periodic[a]) u[a] = (u[a] + nside) & (nside - 1);
      else return 0ull;  // clipped at an open face
    }
  }
  const uint64_t ck = morton3((uint32_t)u[0], (uint32_t)u[1], (uint32_t)u[2]);  // level-L cell key
  int b0, b1;  // bins [b0, b1] covered by the cell
  if (L >= lb) {
    b0 = b1 = (int)(ck >> (3 * (L - lb)));
  } else {
    b0 = (int)(ck << (3 * (lb - L)));
    b1 = (int)(((ck + 1) << (3 * (lb - L))) - 1);
  }
  const int r0 = owner_of_bin(s, world, b0), r1 = owner_of_bin(s, world, b1);
  uint64_t m = 0;
  for (int r = r0; r <= r1; ++r) m |= 1ull << r;
  return m;
}

cudaError_t launch_decomp_ghosts(int64_t n, const uint64_t* key, int bits, int rank, int world,
                                 const int32_t* splits, const DevScalars* ds, const Params& P, uint64_t* mask,
                                 int64_t* counts, cudaStream_t st) {
  cudaError_t e = cudaMemsetAsync(counts, 0, sizeof(int64_t) * world, st);
  if (e != cudaSuccess || n == 0) return e;
  ghost_route_kernel<<<(unsigned)div_up(n, 256), 256, 0, st>>>(n, key, bits, rank, world, splits, ds, P, mask,
                                                               (unsigned long long*)counts);
  note_launch();
  return cudaGetLastError();
}

// ---- rows of every (particle i, destination r in mask[i]), grouped by r in
// rank order, particle order within a destination (deterministic: block counts,
// one scan in (r, block) order, warp ballots).  pos[e] = i of row e.
constexpr int kPackThreads = 1024;

__global__ void __launch_bounds__(kPackThreads) route_count_kernel(int64_t n, const uint64_t* __restrict__ mask,
                                                                   int world, int64_t nb,
                                                                   int64_t* __restrict__ cnt /* [world][nb] */) {
  __shared__ int wc[kMaxGhostRanks][kPackThreads / 32];
  const int64_t i = blockIdx.x * (int64_t)kPackThreads + threadIdx.x;
  const uint64_t m = i < n ? mask[i] : 0ull;
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  for (int r = 0; r < world; ++r) {
    const uint32_t b = __ballot_sync(0xffffffffu, (m >> r) & 1ull);
    if (lane == 0) wc[r][warp] = __popc(b);
  }
  __syncthreads();
  for (int r = threadIdx.x; r < world; r += kPackThreads) {
    int s = 0;
    for (int w = 0; w < kPackThreads / 32; ++w) s += wc[r][w];
    cnt[(int64_t)r * nb + blockIdx.x] = s;
  }
}

__global__ void __launch_bounds__(kPackThreads) route_pack_kernel(int64_t n, const uint64_t* __restrict__ mask,
                                                                  int world, int64_t nb,
                                                                  const int64_t* __restrict__ off /* [world][nb] */,
                                                                  StatePtrs S, const int64_t* __restrict__ id,
                                                                  uint64_t or_id, double* __restrict__ rows,
                                                                  int64_t* __restrict__ pos) {
  __shared__ int wo[kMaxGhostRanks][kPackThreads / 32];
  const int64_t i = blockIdx.x * (int64_t)kPackThreads + threadIdx.x;
  const uint64_t m = i < n ? mask[i] : 0ull;
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  for (int r = 0; r < world; ++r) {
    const uint32_t b = __ballot_sync(0xffffffffu, (m >> r) & 1ull);
    if (lane == 0) wo[r][warp] = __popc(b);
  }
  __syncthreads();
  for (int r = threadIdx.x; r < world; r += kPackThreads) {
    int run = 0;
    for (int w = 0; w < kPackThreads / 32; ++w) {
      const int c = wo[r][w];
      wo[r][w] = run;
      run += c;
    }
  }
  __syncthreads();
  const uint32_t below = (1u << lane) - 1u;
  for (int r = 0; r < world; ++r) {  // uniform loop: every lane takes part in the ballots
    const bool has = (m >> r) & 1ull;
    const uint32_t b = __ballot_sync(0xffffffffu, has);
    if (has) {
      const int64_t e = off[(int64_t)r * nb + blockIdx.x] + wo[r][warp] + __popc(b & below);
      double* row = rows + e * kRowDoubles;
#pragma unroll
      for (int f = 0; f < kNumStateF; ++f) row[f] = S.src[f][i];
      row[kNumStateF] = __longlong_as_double((long long)((uint64_t)id[i] | or_id));
      pos[e] = i;
    }
  }
}

cudaError_t launch_route_pack(int64_t n, const uint64_t* mask, int world, double* const* src, const int64_t* id,
                              uint64_t or_id, double* rows, int64_t* pos, int64_t* scratch, int64_t* total,
                              cudaStream_t st) {
  const int64_t nb = div_up(n, kPackThreads);
  if (n == 0) return cudaMemsetAsync(total, 0, sizeof(int64_t), st);
  route_count_kernel<<<(unsigned)nb, kPackThreads, 0, st>>>(n, mask, world, nb, scratch);
  compact_scan_kernel<<<1, 1024, 0, st>>>(nb * world, scratch, total);  // exclusive, (r, block) order
  StatePtrs S;
  for (int f = 0; f < kNumStateF; ++f) {
    S.src[f] = src[f];
    S.dst[f] = nullptr;
  }
  route_pack_kernel<<<(unsigned)nb, kPackThreads, 0, st>>>(n, mask, world, nb, scratch, S, id, or_id, rows, pos);
  note_launch(3);
  return cudaGetLastError();
}

// ---- positions through the last sort: post[k] = inv[pre[k]] (pre == NULL:
// pre[k] = first + k), inv = the inverse of the sort's permutation
__global__ void __launch_bounds__(256) inverse_perm_kernel(int64_t n, const uint32_t* __restrict__ perm,
                                                           uint32_t* __restrict__ inv) {
  const int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (k < n) inv[perm[k]] = (uint32_t)k;
}

__global__ void __launch_bounds__(256) map_positions_kernel(int64_t m, const int64_t* __restrict__ pre, int64_t first,
                                                            const uint32_t* __restrict__ inv,
                                                            int64_t* __restrict__ post) {
  const int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (k < m) post[k] = inv[pre ? pre[k] : first + k];
}

cudaError_t launch_inverse_perm(int64_t n, const uint32_t* perm, uint32_t* inv, cudaStream_t st) {
  if (n == 0) return cudaSuccess;
  inverse_perm_kernel<<<(unsigned)div_up(n, 256), 256, 0, st>>>(n, perm, inv);
  note_launch();
  return cudaGetLastError();
}

cudaError_t launch_map_positions(int64_t m, const int64_t* pre, int64_t first, const uint32_t* inv, int64_t* post,
                                 cudaStream_t st) {
  if (m == 0) return cudaSuccess;
  map_positions_kernel<<<(unsigned)div_up(m, 256), 256, 0, st>>>(m, pre, first, inv, post);
  note_launch();
  return cudaGetLastError();
}

// ---- halo values: rows [m][nf] of the listed fields at idx (gather) / into
// the listed fields at idx (scatter)
struct FieldList {
  double* f[16];
  int nf;
};

__global__ void __launch_bounds__(256) halo_gather_kernel(int64_t m, const int64_t* __restrict__ idx, FieldList F,
                                                          double* __restrict__ dst) {
  const int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (k >= m) return;
  const int64_t i = idx[k];
  for (int q = 0; q < F.nf; ++q) dst[k * F.nf + q] = F.f[q][i];
}

__global__ void __launch_bounds__(256) halo_scatter_kernel(int64_t m, const int64_t* __restrict__ idx, FieldList F,
                                                           const double* __restrict__ src) {
  const int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (k >= m) return;
  const int64_t i = idx[k];
  for (int q = 0; q < F.nf; ++q) F.f[q][i] = src[k * F.nf + q];
}

cudaError_t launch_halo(int64_t m, const int64_t* idx, double* const* f, int nf, double* buf, bool gather,
                        cudaStream_t st) {
  if (m == 0) return cudaSuccess;
  FieldList F;
  F.nf = nf;
  for (int q = 0; q < nf; ++q) F.f[q] = f[q];
  if (gather) halo_gather_kernel<<<(unsigned)div_up(m, 256), 256, 0, st>>>(m, idx, F, buf);
  else halo_scatter_kernel<<<(unsigned)div_up(m, 256), 256, 0, st>>>(m, idx, F, buf);
  note_launch();
  return cudaGetLastError();
}

}  // namespace sph
