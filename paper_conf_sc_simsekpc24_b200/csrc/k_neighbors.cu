// k_neighbors.cu -- phases CELLS and NEIGHBORS (items 3-4 of DESIGN.md section 3).
//
// CELLS: a uniform grid whose cells are exactly the level-L octree nodes of the
// Morton curve, so every cell is one contiguous range of the sorted particles:
// cell_start[c] .. cell_start[c+1], c = key >> 3(21-L).  Two levels are used: a
// coarse level Lc (the finest with cell side >= 2 h_max on every axis, so a
// target's neighbours lie in the 27 coarse cells around it) and the fine table
// level Lf = Lc + 1 (each coarse cell = 8 consecutive fine cells).  Lc is decided
// on the device from the exact h_max of phase KEYS (no host round trip).
// HBM-bound: 8 B/particle read (key) + 4 B/fine cell written.
//
// NEIGHBORS: warp-cooperative.  A warp takes 32 consecutive (Morton-sorted)
// targets, which sit in a small region of space, and walks ONE candidate stream
// for all of them (no per-lane divergence):
//  1. the coarse cells covering the targets' 2h spheres (<= 128 cells; periodic
//     wrap, clipped at open faces) are ranked by Morton index, so the stream is in
//     ascending particle index -- every lane's neighbours come out ascending, the
//     oracle's order.  A warp whose targets straddle a large Morton jump (box >
//     128 cells) is split into halves, quarters, ... processed one after another;
//  2. per coarse cell, the fine children no lane's sphere reaches are culled
//     (warp OR of per-lane masks); the runs of needed children form a run list
//     (cell_start loads issued by all lanes in parallel, warp prefix sum);
//  3. the runs are streamed 32 candidates at a time (one coalesced 128-bit pos4
//     load per lane, prefetched one chunk ahead, staged in shared memory) and every
//     lane tests every candidate two at a time with packed f32x2 arithmetic
//     (FADD2/FFMA2) against an outer and an inner radius that bracket 2h_i by a
//     rigorous bound on the fp32 rounding (reading 14),
//     the two comparisons taken as the sign bits of packed differences gathered
//     four at a time by PRMT (candidates staged in a permuted slot order so
//     that bit c of the masks is candidate c):
//     outside -> rejected, inside -> accepted; only the thin shell in between
//     (~1e-4 of candidates) runs the oracle's exact fp64 predicate (raw
//     difference, conditional +-L, d2 = (dx*dx + dy*dy) + dz*dz rounded per
//     operation, d2 < (2h_i)(2h_i)).  Every decision equals the exact predicate's:
//     the neighbour sets are bit-identical to brute force;
//  4. each lane appends its own hits, in candidate order, two per iteration and
//     branch-free (a spare word past ngmax absorbs over-capacity stores), to its
//     row-major scratch row (the scratch of the resident CTAs, ~70 MB, mostly
//     stays in L2); when a warp has finished
// its targets, every lane copies its row to the column-major list nbr[k*cap + i]
// (one 128-B line per store instruction) that the neighbour sums read.  The
// kernel is persistent (a grid of SMs x resident CTAs, so the scratch is indexed
// by blockIdx and warp); each warp takes 32-target tiles from an atomic counter,
// in order (dynamic schedule: no tail imbalance, adjacent tiles run together).
// Bound: issue (fp32 + integer work per candidate test, ~880 candidates per
// warp of 32 targets at 100 neighbours).  Algorithmic bytes: pos4, x, y, z, h in
// (48 B), nc out (4 B), the list out (4 B per neighbour).
#include <algorithm>

#include "sph_internal.cuh"

namespace sph {

__global__ void cell_level_kernel(DevScalars* ds, int level_cap) {
  double hmax = unord(ds->hmax_ord);
  int L = level_cap - 1;  // coarse level; the table is one level finer
  while (L > 0) {
    bool ok = true;
    for (int a = 0; a < 3; ++a) {
      double side = (ds->box_max[a] - ds->box_min[a]) / (double)(1 << L);
      if (!(side >= 2.0 * hmax * (1.0 + 1e-9))) ok = false;
    }
    if (ok) break;
    --L;
  }
  ds->cell_level = L + 1;
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
  cell_level_kernel<<<1, 1, 0, st>>>(F.ds, level_cap);
  note_launch();
  if (F.n > 0) {
    cells_kernel<<<(unsigned)div_up(F.n, 256), 256, 0, st>>>(F.n, F.key, F.ds, F.cell_start);
    note_launch();
  }
}

// L2 residency of the scratch rows (SPH_NBR_EVICT): the column-major list
// stores stream 3.2 GB through L2 with evict_first priority, the rows are
// written and read back with evict_last, so the rows are not evicted (and
// written to DRAM and read back) between the appends and the copy-out.
#ifndef SPH_NBR_EVICT
#define SPH_NBR_EVICT 1
#endif
struct L2Pol {
  uint64_t first, last;
};
__device__ __forceinline__ L2Pol make_l2pol() {
  L2Pol p{0, 0};
  if (SPH_NBR_EVICT) {
    asm("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p.first));
    asm("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(p.last));
  }
  return p;
}
__device__ __forceinline__ void st_hint(int32_t* a, int32_t v, uint64_t pol) {
  if (SPH_NBR_EVICT) asm volatile("st.global.L2::cache_hint.b32 [%0], %1, %2;" ::"l"(a), "r"(v), "l"(pol) : "memory");
  else *a = v;
}
__device__ __forceinline__ void ld8i_hint(const int32_t* p, int (&v)[8], uint64_t pol) {
  if (SPH_NBR_EVICT)
    asm volatile("ld.global.L2::cache_hint.v8.b32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8], %9;"
                 : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7])
                 : "l"(p), "l"(pol)
                 : "memory");
  else
    ld8i(p, v);
}

constexpr int kNbrThreads = 128;
#ifndef SPH_NBR_MINB
#define SPH_NBR_MINB 6  // resident CTAs per SM (6 -> 80 registers)
#endif
constexpr int kNbrWarps = kNbrThreads / 32;
constexpr int kMaxWarpCells = 128;

// Per-target constants of the search.
struct Target {
  double x, y, z, r2max;  // fp64 position and (2h)^2 for the exact predicate
  float m[3];             // fp32 position relative to box_min
  float r_out2, r_in2;    // fp32 bracket of (2h)^2
  float rc;               // culling radius
};

struct Box {
  double L[3], H[3];
  float Lf[3], side[3];    // box length, coarse cell side (fp32)
  bool per[3];
  int nside;               // coarse cells per axis
  int Lc;
};

__device__ __forceinline__ Target make_target(const Fields& F, const Box& B, int64_t i, bool active) {
  Target t;
  if (!active) {
    t.x = t.y = t.z = 0.0;
    t.r2max = -1.0;
    t.m[0] = t.m[1] = t.m[2] = 0.f;
    t.r_out2 = -1.f;  // rejects every candidate
    t.r_in2 = -1.f;
    t.rc = -1.f;
    return t;
  }
  t.x = F.f[FX][i];
  t.y = F.f[FY][i];
  t.z = F.f[FZ][i];
  const double h = F.f[FH][i];
  const double r = 2.0 * h;
  t.r2max = r * r;
  const double Lmax = fmax(B.L[0], fmax(B.L[1], B.L[2]));
  // fp32 rounding bound per axis: pos4 conversion, shift by +-L and the
  // difference each add <= 2^-24 L  ->  E = 8 * 2^-24 * L (reading 14)
  const double E = 8.0 * 5.9604644775390625e-08 * Lmax;
  const double sE = 1.7320508075688772 * E;
  t.r_out2 = __double2float_ru((r + sE) * (r + sE) * (1.0 + 1e-6));
  t.r_in2 = r > sE ? __double2float_rd((r - sE) * (r - sE) * (1.0 - 1e-6)) : -1.0f;
  t.rc = __double2float_ru((r + sE + 4.0 * E) * (1.0 + 1e-6));
  const float4 me = F.pos4[i];
  t.m[0] = me.x;
  t.m[1] = me.y;
  t.m[2] = me.z;
  return t;
}

// The exact predicate of item 4 (only reached for the thin fp32 shell).
__device__ __forceinline__ bool exact_in(const Fields& F, const Box& B, const Target& t, uint32_t j) {
  double ex = min_image(__dsub_rn(t.x, F.f[FX][j]), B.L[0], B.H[0], B.per[0]);
  double ey = min_image(__dsub_rn(t.y, F.f[FY][j]), B.L[1], B.H[1], B.per[1]);
  double ez = min_image(__dsub_rn(t.z, F.f[FZ][j]), B.L[2], B.H[2], B.per[2]);
  return __dadd_rn(__dadd_rn(__dmul_rn(ex, ex), __dmul_rn(ey, ey)), __dmul_rn(ez, ez)) < t.r2max;
}

// Per-axis squared distances from the target to the lower/upper child slab of
// the coarse cell at unwrapped coordinate u (0 when the axis is "full": the
// warp's range covers the whole periodic axis and the image is resolved per
// candidate).
__device__ __forceinline__ void slab_d2(const Box& B, const Target& t, int a, int u, bool full,
                                        float& d0, float& d1) {
  if (full) {
    d0 = d1 = 0.f;
    return;
  }
  const float lo = (float)u * B.side[a];
  const float half = 0.5f * B.side[a];
  const float m = t.m[a];
  float a0 = fmaxf(fmaxf(lo - m, m - (lo + half)), 0.f);
  float a1 = fmaxf(fmaxf(lo + half - m, m - (lo + B.side[a])), 0.f);
  d0 = a0 * a0;
  d1 = a1 * a1;
}

// Packed fp32x2 arithmetic: pack2 / sub2 / mul2 / fma2 (sph_internal.cuh).

// Run table size.  A cell contributes up to 4 runs of needed children; when the
// group's runs would exceed kMaxRuns, each cell's needed children are merged into
// one run (the unneeded children in between become candidates that fail the
// test), so kMaxRuns >= kMaxWarpCells always suffices.  A small table leaves
// more of the SM's 256 KB to L1.
// 1: a chunk's candidates find their runs by one warp mask of the run starts in
// the chunk; 0: each lane advances its own run pointer (a divergent loop).
#ifndef SPH_NBR_RUNSCAN
#define SPH_NBR_RUNSCAN 1
#endif
#ifndef SPH_NBR_DISCARD
#define SPH_NBR_DISCARD 0  // A/B: DRAM writes 4.51 -> 3.72 GB, time 7.13 -> 7.24 ms
#endif
#ifndef SPH_NBR_IMGSKIP
#define SPH_NBR_IMGSKIP 1
#endif
#ifndef SPH_NBR_MAXRUNS
#define SPH_NBR_MAXRUNS 128
#endif
constexpr int kMaxRuns = SPH_NBR_MAXRUNS;
static_assert(kMaxRuns >= kMaxWarpCells, "one merged run per cell must fit");

struct WarpSmem {
  uint32_t cell[kMaxWarpCells];   // sorted coarse cell keys
  uint32_t ucs[kMaxWarpCells];    // their unwrapped coordinates (biased, packed)
  uint32_t mask[kMaxWarpCells];   // children any lane needs
  union {
    struct {
      uint32_t run_start[kMaxRuns];   // first particle of each run
      uint32_t run_pos[kMaxRuns + 1]; // stream position of each run (exclusive prefix)
      uint32_t run_cell[kMaxRuns];    // periodic image code of the run's cell (2 bits/axis)
    };
    unsigned long long sortkey[kMaxWarpCells];  // build_cells scratch
  };
  // staged chunk of 32 candidates (image-shifted fp32 position, SoA so that two
  // consecutive candidates are one 64-bit load for the packed f32x2 math)
  alignas(16) float cx[32];
  alignas(16) float cy[32];
  alignas(16) float cz[32];
  uint32_t cj[32];
  uint32_t selfm[32];             // per target: chunk slots holding the target itself
};

// The group's coarse cells: T distinct (wrapped key, unwrapped coordinates)
// entries, sorted, in WarpSmem::cell / ::ucs.  "full" axes are periodic axes
// with fewer than 3 coarse cells: there images are resolved per candidate
// (minimum image in fp32) and every entry is its own wrapped cell.
struct GroupBox {
  bool full[3];
  int T;
};

// Builds the sorted union of the 27-cell stencils of the group's distinct
// coarse cells (at most kMaxGroupCells of them, leader lanes in `leaders`).
// Entries for the same wrapped cell reached through different periodic images
// are kept apart (each target uses exactly one image of any particle).
constexpr int kMaxGroupCells = 4;  // 4 x 27 = 108 <= kMaxWarpCells stencil entries

__device__ __forceinline__ GroupBox build_cells(const Box& B, const int (&cc)[3], uint32_t leaders,
                                                int lane, WarpSmem& S) {
  GroupBox G;
  const int n = B.nside, nm = n - 1;
#pragma unroll
  for (int a = 0; a < 3; ++a) G.full[a] = B.per[a] && n < 3;
  const int D = __popc(leaders);
  // the leaders' coarse coordinates, broadcast
  int lc[kMaxGroupCells][3];
  {
    uint32_t l = leaders;
#pragma unroll
    for (int d = 0; d < kMaxGroupCells; ++d) {
      const int src = l ? __ffs(l) - 1 : 0;
      if (l) l &= l - 1;
#pragma unroll
      for (int a = 0; a < 3; ++a) lc[d][a] = __shfl_sync(0xffffffffu, cc[a], src);
    }
  }
  // stencil entries, 4 per lane: 64-bit sort key (wrapped key << 30 | packed unwrapped)
  unsigned long long v[kMaxWarpCells / 32];
#pragma unroll
  for (int r = 0; r < kMaxWarpCells / 32; ++r) {
    const int e = r * 32 + lane;
    v[r] = ~0ull;
    if (e < D * 27) {
      int d = e / 27, s = e - d * 27;
      int base[3] = {lc[0][0], lc[0][1], lc[0][2]};
#pragma unroll
      for (int q = 1; q < kMaxGroupCells; ++q)
        if (d == q) {
          base[0] = lc[q][0];
          base[1] = lc[q][1];
          base[2] = lc[q][2];
        }
      const int o[3] = {s / 9 - 1, (s / 3) % 3 - 1, s % 3 - 1};
      int u[3];
      bool ok = true;
#pragma unroll
      for (int a = 0; a < 3; ++a) {
        u[a] = base[a] + o[a];
        if (G.full[a]) u[a] &= nm;                         // one entry per wrapped cell
        else if (!B.per[a] && (u[a] < 0 || u[a] >= n)) ok = false;  // open face
      }
      if (ok) {
        const uint64_t key = morton3((uint32_t)(u[0] & nm), (uint32_t)(u[1] & nm), (uint32_t)(u[2] & nm));
        const uint32_t pk = (uint32_t)(u[0] + 4) | ((uint32_t)(u[1] + 4) << 10) | ((uint32_t)(u[2] + 4) << 20);
        v[r] = (key << 30) | pk;
      }
    }
  }
  // rank sort (ties -> lower slot first), then drop duplicates
  unsigned long long* sk = S.sortkey;
#pragma unroll
  for (int r = 0; r < kMaxWarpCells / 32; ++r) sk[r * 32 + lane] = v[r];
  __syncwarp();
  uint32_t rank[kMaxWarpCells / 32] = {0, 0, 0, 0};
  const int E = D * 27;
  // only the registers that hold entries are ranked (E = 27 for the common
  // one-cell group: one compare per entry instead of four)
  if (E <= 32) {
    for (int u = 0; u < E; ++u) {
      const unsigned long long w = sk[u];
      rank[0] += (w < v[0] || (w == v[0] && u < lane)) ? 1u : 0u;
    }
  } else if (E <= 64) {
    for (int u = 0; u < E; ++u) {
      const unsigned long long w = sk[u];
#pragma unroll
      for (int r = 0; r < 2; ++r) rank[r] += (w < v[r] || (w == v[r] && u < r * 32 + lane)) ? 1u : 0u;
    }
  } else {
    for (int u = 0; u < E; ++u) {
      const unsigned long long w = sk[u];
#pragma unroll
      for (int r = 0; r < kMaxWarpCells / 32; ++r)
        rank[r] += (w < v[r] || (w == v[r] && u < r * 32 + lane)) ? 1u : 0u;
    }
  }
  __syncwarp();
#pragma unroll
  for (int r = 0; r < kMaxWarpCells / 32; ++r)
    if (r * 32 + lane < E) sk[rank[r]] = v[r];
  __syncwarp();
  int T = 0;
#pragma unroll
  for (int r = 0; r < (E + 31) / 32; ++r) {
    const int p = r * 32 + lane;
    const unsigned long long w = p < E ? sk[p] : ~0ull;
    const bool keep = w != ~0ull && (p == 0 || sk[p - 1] != w);
    const uint32_t b = __ballot_sync(0xffffffffu, keep);
    const int pos = T + __popc(b & ((1u << lane) - 1u));
    T += __popc(b);
    __syncwarp();
    if (keep) {
      S.cell[pos] = (uint32_t)(w >> 30);
      S.ucs[pos] = (uint32_t)(w & 0x3fffffffull);
    }
  }
  __syncwarp();
  G.T = T;
  return G;
}

// The group's candidate stream (see the file header, steps 2-4).  Lanes with
// t.rc < 0 take part in the warp collectives but test nothing.
template <bool kFull>
__device__ __forceinline__ void warp_walk(const Fields& F, const Box& B, const Target& t, int64_t i,
                                          const GroupBox& G, WarpSmem& S, int lane, int& cnt,
                                          bool& bnd, int32_t* __restrict__ rows, const L2Pol& pol,
                                          int merge_runs) {
  const int n = B.nside;
  const int T = G.T;
  const int ngmax = F.ngmax;
  const float rc2 = t.rc * t.rc;
  const bool live = t.rc >= 0.f;
  // ---- 2a. needed children per cell (warp OR)
  for (int u = 0; u < T; ++u) {
    const uint32_t pk = S.ucs[u];
    const int uc[3] = {(int)(pk & 1023u) - 4, (int)((pk >> 10) & 1023u) - 4, (int)(pk >> 20) - 4};
    float d[3][2];
#pragma unroll
    for (int a = 0; a < 3; ++a) slab_d2(B, t, a, uc[a], kFull && G.full[a], d[a][0], d[a][1]);
    uint32_t mask = 0;
#pragma unroll
    for (int b = 0; b < 8; ++b)
      if (live && d[0][b >> 2] + d[1][(b >> 1) & 1] + d[2][b & 1] <= rc2) mask |= 1u << b;
    mask = __reduce_or_sync(0xffffffffu, mask);
    if (lane == 0) S.mask[u] = mask;
  }
  __syncwarp();
  // ---- 2b. runs (one cell per lane), placed by a warp prefix sum in cell order
  bool img = false;    // any run of a periodic image cell (shifted candidates)
  bool merge = false;  // one run per cell (see kMaxRuns)
  const int run_lim = merge_runs < 0 ? kMaxRuns : min(merge_runs, kMaxRuns);
  if (4 * T > run_lim) {
    uint32_t tr = 0;
    for (int u = lane; u < T; u += 32) {
      const uint32_t mk = S.mask[u];
      tr += __popc(mk & ~(mk << 1));  // runs of set bits
    }
    merge = __reduce_add_sync(0xffffffffu, tr) > (uint32_t)run_lim;
  }
  uint32_t nruns = 0, ncand = 0;
  for (int r0 = 0; r0 < T; r0 += 32) {
    const int u = r0 + lane;
    const uint32_t mask = u < T ? S.mask[u] : 0u;
    uint32_t bnd[9];
#pragma unroll
    for (int b = 0; b < 9; ++b) bnd[b] = 0;
    if (mask) {
      const uint32_t* cs = F.cell_start + ((size_t)S.cell[u] << 3);
#pragma unroll
      for (int b = 0; b < 9; ++b) bnd[b] = cs[b];
    }
    uint32_t my_runs = 0, my_cand = 0;
    uint32_t rs[4], re[4];
#pragma unroll
    for (int q = 0; q < 4; ++q) rs[q] = re[q] = 0;
    uint32_t m = mask;
    if (merge && mask) m = ((2u << (31 - __clz(mask))) - 1u) & ~((1u << (__ffs(mask) - 1)) - 1u);
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      if (m) {
        const int b0 = __ffs(m) - 1;
        const uint32_t run = (~(m >> b0)) & 0xffu;  // first zero bit above the run
        const int b1 = b0 + (run ? __ffs(run) - 1 : 8 - b0);
        m &= ~(((1u << b1) - 1u) & ~((1u << b0) - 1u));
        uint32_t j0 = 0, j1 = 0;
#pragma unroll
        for (int b = 0; b < 9; ++b) {
          j0 = (b == b0) ? bnd[b] : j0;
          j1 = (b == b1) ? bnd[b] : j1;
        }
        if (j1 > j0) {
          rs[my_runs] = j0;
          re[my_runs] = j1;
          my_cand += j1 - j0;
          ++my_runs;
        }
      }
    }
    uint32_t sr = my_runs, sc = my_cand;
#pragma unroll
    for (int off = 1; off < 32; off <<= 1) {
      const uint32_t a1 = __shfl_up_sync(0xffffffffu, sr, off), a2 = __shfl_up_sync(0xffffffffu, sc, off);
      if (lane >= off) {
        sr += a1;
        sc += a2;
      }
    }
    uint32_t pr = nruns + sr - my_runs, pc = ncand + sc - my_cand;
    // periodic image of this cell: per axis 0 (inside), 1 (u < 0: stored one box
    // length above), 2 (u >= n: stored one box length below)
    uint32_t code = 0;
    if (my_runs) {
      const uint32_t pk = S.ucs[u];
      const int uc[3] = {(int)(pk & 1023u) - 4, (int)((pk >> 10) & 1023u) - 4, (int)(pk >> 20) - 4};
#pragma unroll
      for (int a = 0; a < 3; ++a)
        if (!(kFull && G.full[a])) code |= (uint32_t)(uc[a] < 0 ? 1 : (uc[a] >= n ? 2 : 0)) << (2 * a);
    }
    img = img || __any_sync(0xffffffffu, code != 0u);
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      if (q < (int)my_runs) {
        S.run_start[pr + q] = rs[q];
        S.run_pos[pr + q] = pc;
        S.run_cell[pr + q] = code;
        pc += re[q] - rs[q];
      }
    }
    nruns += __shfl_sync(0xffffffffu, sr, 31);
    ncand += __shfl_sync(0xffffffffu, sc, 31);
  }
  if (lane == 0) {
    S.run_pos[nruns] = ncand;
    atomicAdd(&F.ds->cand_total, (unsigned long long)ncand);  // diagnostics
    atomicAdd(&F.ds->pass_total, 1ull);
  }
  __syncwarp();

  // ---- 3./4. stream, test, append
  const uint32_t nchunks = (ncand + 31) / 32;
  uint32_t run = 0;
#if SPH_NBR_RUNSCAN
  int rb = -1;  // warp-uniform: the last run starting before the chunk
#endif
  float4 q = make_float4(__int_as_float(0x7fc00000), 0.f, 0.f, 0.f);  // NaN: fails every test
  float sx = 0.f, sy = 0.f, sz = 0.f;
  uint32_t qj = 0;
  auto load = [&](uint32_t c) {
    const uint32_t g = c * 32 + (uint32_t)lane;
#if SPH_NBR_RUNSCAN
    {
      // each lane examines one of the next 32 run starts; the runs starting in
      // this chunk become bits of a warp mask, and a lane's run is the number of
      // starts at or below its slot (no per-lane search loop)
      const int e = rb + 1 + lane;
      const uint32_t st = e <= (int)nruns ? S.run_pos[e] : 0xffffffffu;
      const uint32_t off = st - c * 32;  // >= 0: run rb + 1 starts after the previous chunk
      const uint32_t smask = __reduce_or_sync(0xffffffffu, off < 32u ? 1u << off : 0u);
      run = (uint32_t)(rb + __popc(smask & ((2u << lane) - 1u)));
      rb += __popc(smask);
    }
#endif
    sx = sy = sz = 0.f;
    if (g >= ncand) {
      q = make_float4(__int_as_float(0x7fc00000), 0.f, 0.f, 0.f);
      qj = 0;
      return;
    }
#if !SPH_NBR_RUNSCAN
    while (S.run_pos[run + 1] <= g) ++run;
#endif
    qj = S.run_start[run] + (g - S.run_pos[run]);
    q = F.pos4[qj];
    // unwrapped position of the candidate = stored + k L (k = -1, 0, 1); the
    // shift is applied when the chunk is staged (keeps the load latency hidden).
    // Most warps have no image cell at all (warp-uniform skip).
    if (SPH_NBR_IMGSKIP && !img) return;
    const uint32_t code = S.run_cell[run];
    const uint32_t c0 = code & 3u, c1 = (code >> 2) & 3u, c2 = (code >> 4) & 3u;
    sx = c0 == 1u ? -B.Lf[0] : (c0 == 2u ? B.Lf[0] : 0.f);
    sy = c1 == 1u ? -B.Lf[1] : (c1 == 2u ? B.Lf[1] : 0.f);
    sz = c2 == 1u ? -B.Lf[2] : (c2 == 2u ? B.Lf[2] : 0.f);
  };
  const unsigned long long mx2 = pack2(t.m[0], t.m[0]), my2 = pack2(t.m[1], t.m[1]),
                           mz2 = pack2(t.m[2], t.m[2]);
  const int64_t wbase = i - lane;  // the warp's first target
  S.selfm[lane] = 0u;
  if (nchunks) load(0);
  // candidate c is staged at slot sigma(c) = 4 (c & 7) + (c >> 3): the sign-bit
  // gathering below then yields bit c for candidate c
  const int sg = 4 * (lane & 7) + (lane >> 3);
  const unsigned long long rin2x2 = pack2(t.r_in2, t.r_in2), rout2x2 = pack2(t.r_out2, t.r_out2);
  for (uint32_t c = 0; c < nchunks; ++c) {
    const uint32_t gmask = __ballot_sync(0xffffffffu, q.w != 0.f);  // candidates that are ghosts
    S.cx[sg] = q.x + sx;
    S.cy[sg] = q.y + sy;
    S.cz[sg] = q.z + sz;
    S.cj[lane] = qj;
    if (c * 32 + (uint32_t)lane < ncand && (uint64_t)((int64_t)qj - wbase) < 32u)
      atomicOr(&S.selfm[(int64_t)qj - wbase], 1u << lane);  // candidate is a target of this warp
    __syncwarp();
    if (c + 1 < nchunks) load(c + 1);
    uint32_t hin = 0, hout = 0;
    uint32_t pin_prev = 0, pout_prev = 0;
#pragma unroll
    for (int k = 0; k < 32; k += 2) {
      const unsigned long long px = *reinterpret_cast<const unsigned long long*>(&S.cx[k]);
      const unsigned long long py = *reinterpret_cast<const unsigned long long*>(&S.cy[k]);
      const unsigned long long pz = *reinterpret_cast<const unsigned long long*>(&S.cz[k]);
      unsigned long long dx = sub2(mx2, px), dy = sub2(my2, py), dz = sub2(mz2, pz);
      if (kFull) {
        float a0, a1;
        unpack2(dx, a0, a1);
        if (G.full[0]) { a0 -= B.Lf[0] * rintf(a0 / B.Lf[0]); a1 -= B.Lf[0] * rintf(a1 / B.Lf[0]); }
        dx = pack2(a0, a1);
        unpack2(dy, a0, a1);
        if (G.full[1]) { a0 -= B.Lf[1] * rintf(a0 / B.Lf[1]); a1 -= B.Lf[1] * rintf(a1 / B.Lf[1]); }
        dy = pack2(a0, a1);
        unpack2(dz, a0, a1);
        if (G.full[2]) { a0 -= B.Lf[2] * rintf(a0 / B.Lf[2]); a1 -= B.Lf[2] * rintf(a1 / B.Lf[2]); }
        dz = pack2(a0, a1);
      }
      const unsigned long long d2 = fma2(dx, dx, fma2(dy, dy, mul2(dz, dz)));
      // d2 < r  <=>  sign(fl(d2 - r)) (exact: a rounded difference keeps the sign
      // and is +0 only for d2 == r; canonical NaN is positive).  The sign bytes
      // of 4 slots are gathered by PRMT, then shifted into bit positions.
      const unsigned long long din = sub2(d2, rin2x2), dout = sub2(d2, rout2x2);
      const uint32_t pin = __byte_perm((uint32_t)din, (uint32_t)(din >> 32), 0x0073);
      const uint32_t pout = __byte_perm((uint32_t)dout, (uint32_t)(dout >> 32), 0x0073);
      if ((k & 2) == 0) {
        pin_prev = pin;
        pout_prev = pout;
      } else {
        const int gq = k >> 2;
        hin |= (__byte_perm(pin_prev, pin, 0x5410) >> (7 - gq)) & (0x01010101u << gq);
        hout |= (__byte_perm(pout_prev, pout, 0x5410) >> (7 - gq)) & (0x01010101u << gq);
      }
    }
    // thin shell: the exact fp64 predicate decides (rare)
    uint32_t shell = hout & ~hin;
    if (__any_sync(0xffffffffu, shell != 0)) {
      while (shell) {
        const int k = __ffs(shell) - 1;
        shell &= shell - 1;
        if (exact_in(F, B, t, S.cj[k])) hin |= 1u << k;
      }
    }
    // the target itself (d = 0) is not its own neighbour
    hin &= ~S.selfm[lane];
    bnd = bnd || (hin & gmask) != 0u;
    // append: every lane writes its own hits, in candidate (= ascending index)
    // order, to its L2-resident row.  The warp runs the busiest lane's
    // iterations (~8-12 per chunk), but each is 5 instructions; a cooperative
    // append (owner by binary search over the prefix of hit counts, r-th hit by
    // a popc search, few lines per store) was 9.85 vs 9.07 ms: its shuffle
    // chains cost more than the scattered row stores.
    const int pc = __popc(hin);
    {
      uint32_t m = hin;
      int slot = cnt;
      int32_t* myrow = rows + lane * F.nrows_ld;
      // two hits per iteration (the warp runs the busiest lane's count)
      while (m) {
        const int b0 = __ffs(m) - 1;
        m &= m - 1;
        const int b1 = m ? __ffs(m) - 1 : b0;
        const bool two = m != 0;
        m &= m - 1;
        const int32_t v0 = (int32_t)S.cj[b0], v1 = (int32_t)S.cj[b1];
        // branch-free: past the capacity (or for a missing second hit) the
        // store goes to the row's spare word ngmax (nrows_ld > ngmax), never read
        st_hint(myrow + min(slot, ngmax), v0, pol.last);
        st_hint(myrow + (two ? min(slot + 1, ngmax) : ngmax), v1, pol.last);
        slot += two ? 2 : 1;
      }
    }
    cnt += pc;
    S.selfm[lane] = 0u;
    __syncwarp();
  }
}

__global__ void __launch_bounds__(kNbrThreads, SPH_NBR_MINB) neighbors_kernel(Fields F, Params P) {
  __shared__ WarpSmem s_w[kNbrWarps];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const DevScalars* ds = F.ds;
  Box B;
  B.Lc = ds->cell_level - 1;
  B.nside = 1 << B.Lc;
#pragma unroll
  for (int a = 0; a < 3; ++a) {
    B.L[a] = ds->box_max[a] - ds->box_min[a];
    B.H[a] = 0.5 * B.L[a];
    B.Lf[a] = (float)B.L[a];
    B.side[a] = (float)(B.L[a] / B.nside);
    B.per[a] = P.periodic[a] != 0;
  }
  const L2Pol pol = make_l2pol();
  // this warp's 32 scratch rows (row of lane l: rows + l * nrows_ld)
  int32_t* const rows = F.nrows + ((int64_t)blockIdx.x * kNbrThreads + warp * 32) * F.nrows_ld;
  // warps take 32-target tiles dynamically, in order (Morton-adjacent tiles run
  // at about the same time: L2 locality of the candidate data; no tail imbalance)
  while (true) {
    unsigned long long wt = 0;
    if (lane == 0) wt = atomicAdd(&F.ds->nbr_next, 1ull);
    wt = __shfl_sync(0xffffffffu, wt, 0);
    const int64_t i = (int64_t)wt * 32 + lane;
    if ((int64_t)wt * 32 >= F.n) break;
    // ghosts (SPH_GHOST_BIT) are candidates only: no list of their own (nc = 0)
    const bool ghost = i < F.n && (F.id[i] & SPH_GHOST_BIT);
    const bool active = i < F.n && !ghost;
    const Target t = make_target(F, B, i, active);
    int cc[3] = {0, 0, 0};
    uint32_t ckey = 0;
    if (active) {
      const uint64_t key = F.key[i];
      const int sh = 21 - B.Lc;
      cc[0] = (int)(compact3(key >> 2) >> sh);
      cc[1] = (int)(compact3(key >> 1) >> sh);
      cc[2] = (int)(compact3(key) >> sh);
      ckey = (uint32_t)(key >> (3 * sh));
    }
    int cnt = 0;
    bool bnd = false;

    // group size: the whole warp unless it spans more than kMaxGroupCells distinct
    // coarse cells (Morton jumps); then halves, quarters, ...
    int g = 32;
    uint32_t leaders;
    while (true) {
      const unsigned long long tag =
          active ? (((unsigned long long)(lane / g)) << 32) | ckey : (0xffffffff00000000ull | (unsigned)lane);
      const uint32_t peers = __match_any_sync(0xffffffffu, tag);
      const bool lead = active && (peers & ((1u << lane) - 1u)) == 0;
      leaders = __ballot_sync(0xffffffffu, lead);
      const uint32_t gm = (g == 32) ? 0xffffffffu : (((1u << g) - 1u) << ((lane / g) * g));
      const int D = __popc(leaders & gm);
      if (g == 1 || __reduce_max_sync(0xffffffffu, D) <= kMaxGroupCells) break;
      g >>= 1;
    }
    for (int gid = 0; gid < 32 / g; ++gid) {
      const uint32_t gm = (g == 32) ? 0xffffffffu : (((1u << g) - 1u) << (gid * g));
      const uint32_t gl = leaders & gm;
      if (!gl) continue;
      const GroupBox G = build_cells(B, cc, gl, lane, s_w[warp]);
      Target tg = t;
      if (lane / g != gid) tg.r_out2 = tg.r_in2 = tg.rc = -1.f;  // not in this pass
      if (G.full[0] || G.full[1] || G.full[2])
        warp_walk<true>(F, B, tg, i, G, s_w[warp], lane, cnt, bnd, rows, pol, P.nbr_merge_runs);
      else
        warp_walk<false>(F, B, tg, i, G, s_w[warp], lane, cnt, bnd, rows, pol, P.nbr_merge_runs);
      __syncwarp();
    }
    if (active) {
      F.nc[i] = cnt;
      F.bnd[i] = bnd ? 1 : 0;
    } else if (ghost) {
      F.nc[i] = 0;
      F.bnd[i] = 0;
    }
    // copy the rows to the column-major list: lane l holds row l; the store of
    // slot k by the 32 lanes is one 128-B line
    const int len = active ? min(cnt, F.ngmax) : 0;
    const int wlen = __reduce_max_sync(0xffffffffu, len);
    const int32_t* myrow = rows + lane * F.nrows_ld;
    int32_t* col = F.nbr + i;
    for (int k0 = 0; k0 < wlen; k0 += 8) {
      int v[8];
      if (k0 < len) ld8i_hint(myrow + k0, v, pol.last);
#pragma unroll
      for (int u = 0; u < 8; ++u)
        if (k0 + u < len) st_hint(col + (int64_t)(k0 + u) * F.cap, v[u], pol.first);
    }
    __syncwarp();  // the rows are reused by the next tile
#if SPH_NBR_DISCARD
    // the rows are dead: drop their (dirty) L2 lines instead of letting them be
    // written back to DRAM when evicted later (the warp's scratch is nrows_ld
    // whole 128-B lines)
    for (int q = lane; q < (int)F.nrows_ld; q += 32)
      asm volatile("discard.global.L2 [%0], 128;" ::"l"(rows + (int64_t)q * 32) : "memory");
#endif

    // nc statistics (min, max, total) and the capacity flag.
    int mn = active ? cnt : 0x7fffffff, mx = active ? cnt : 0;
    unsigned long long tot = active ? (unsigned long long)cnt : 0ull;
#pragma unroll
    for (int off = 16; off > 0; off >>= 1) {
      mn = min(mn, __shfl_xor_sync(0xffffffffu, mn, off));
      mx = max(mx, __shfl_xor_sync(0xffffffffu, mx, off));
      tot += __shfl_xor_sync(0xffffffffu, tot, off);
    }
    if (lane == 0) {
      atomicMin(&F.ds->min_nc, mn);
      atomicMax(&F.ds->max_nc, mx);
      atomicAdd(&F.ds->total_nc, tot);
      if (mx > F.ngmax) atomicOr(&F.ds->status, (int)ST_CAPACITY);
    }
  }
}

void launch_neighbors(const Fields& F, const Params& P, cudaStream_t st) {
  if (F.n == 0) return;
  static int resident = 0;  // SMs x resident CTAs of this kernel (<= kNbrSlots)
  if (!resident) {
    int dev = 0, sms = 0, per = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, neighbors_kernel, kNbrThreads, 0);
    resident = std::max(1, std::min(kNbrSlots, sms * std::max(per, 1)));
  }
  const int64_t grid = std::min<int64_t>(div_up(F.n, kNbrThreads), resident);
  cudaMemsetAsync(&F.ds->nbr_next, 0, sizeof(unsigned long long), st);
  neighbors_kernel<<<(unsigned)grid, kNbrThreads, 0, st>>>(F, P);
  note_launch();
}

}  // namespace sph
