// k_sort.cu -- phase SORT: stable onesweep LSD radix sort of the 63-bit Morton
// keys (item 3 of DESIGN.md section 3: std::stable_sort by key == LSD radix
// sort with stable passes), 8 passes of 8-bit digits.
//
// Design (one read + one write of (key, index) per pass):
//   1. one histogram kernel reads every key once and builds the 8 per-pass digit
//      histograms (warp-aggregated shared atomics, then global atomics);
//   2. per pass, one kernel: each CTA takes the next tile id from a global
//      counter (so every tile it may wait on is already running: forward
//      progress without co-residency assumptions), ranks its 2048 keys stably
//      with warp match/ballot (per-warp digit counters in shared memory),
//      publishes its digit counts, resolves its global digit offsets by
//      decoupled look-back over the preceding tiles' published words
//      (2 flag bits + 30-bit count in one 32-bit word), reorders the tile in
//      shared memory and writes each digit run out coalesced.
// The first pass generates the index payload (iota) instead of reading it.
//
// Roofline: HBM-bound.  Algorithmic bytes per particle: 8 (histogram read) +
// 8 passes x (8 + 4 read, 8 + 4 write) - 4 (first pass reads no index) = 196 B.
#include <algorithm>

#include "sph_internal.cuh"

namespace sph {

constexpr uint32_t kFlagAgg = 1u << 30;
constexpr uint32_t kFlagInc = 2u << 30;
constexpr uint32_t kValMask = (1u << 30) - 1;
constexpr int kHistThreads = 256;

__device__ __forceinline__ uint32_t ld_relaxed(const uint32_t* p) {
  uint32_t v;
  asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_relaxed(uint32_t* p, uint32_t v) {
  asm volatile("st.relaxed.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ uint32_t lanemask_lt() {
  uint32_t m;
  asm("mov.u32 %0, %%lanemask_lt;" : "=r"(m));
  return m;
}

// All 8 digit histograms in one read of the keys.  Each thread takes 8
// consecutive keys.  The keys arrive nearly sorted (last step's order), so in
// the high-digit passes a thread's 8 digits form one run and a warp's 256 keys
// usually share the digit: runs are counted in registers and a warp whose
// lanes all hold the same single-run digit adds once (warp reduction); the
// low-digit passes (jitter bits, effectively random) add per run.
__global__ void __launch_bounds__(kHistThreads) sort_hist_kernel(const uint64_t* __restrict__ keys,
                                                                 int64_t n, uint32_t* __restrict__ hist) {
  __shared__ uint32_t sh[kSortPasses][kRadix];
  for (int t = threadIdx.x; t < kSortPasses * kRadix; t += blockDim.x) (&sh[0][0])[t] = 0;
  __syncthreads();
  const int64_t nchunks = (n + 7) / 8;
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  // whole warps iterate together (warp collectives below)
  for (int64_t c0 = blockIdx.x * (int64_t)blockDim.x + (threadIdx.x & ~31); c0 < nchunks; c0 += stride) {
    const int64_t c = c0 + (threadIdx.x & 31);
    const int64_t i0 = c * 8;
    const int cnt = c < nchunks ? (int)(n - i0 < 8 ? n - i0 : 8) : 0;
    uint64_t k[8];
#pragma unroll
    for (int j = 0; j < 8; ++j) k[j] = j < cnt ? keys[i0 + j] : 0ull;
#pragma unroll
    for (int p = 0; p < kSortPasses; ++p) {
      const int sh_bits = p * kRadixBits;
      uint32_t prev = (uint32_t)((k[0] >> sh_bits) & (kRadix - 1));
      bool single = true;
#pragma unroll
      for (int j = 1; j < 8; ++j)
        if (j < cnt && (uint32_t)((k[j] >> sh_bits) & (kRadix - 1)) != prev) single = false;
      const uint32_t d0 = __shfl_sync(0xffffffffu, prev, 0);
      if (__all_sync(0xffffffffu, cnt == 0 || (single && prev == d0))) {
        const uint32_t tot = __reduce_add_sync(0xffffffffu, (uint32_t)cnt);
        if ((threadIdx.x & 31) == 0 && tot) atomicAdd(&sh[p][d0], tot);
        continue;
      }
      if (cnt == 0) continue;
      uint32_t run = 1;
#pragma unroll
      for (int j = 1; j < 8; ++j) {
        if (j < cnt) {
          const uint32_t d = (uint32_t)((k[j] >> sh_bits) & (kRadix - 1));
          if (d == prev) {
            ++run;
          } else {
            atomicAdd(&sh[p][prev], run);
            prev = d;
            run = 1;
          }
        }
      }
      atomicAdd(&sh[p][prev], run);
    }
  }
  __syncthreads();
  for (int t = threadIdx.x; t < kSortPasses * kRadix; t += blockDim.x) {
    uint32_t v = (&sh[0][0])[t];
    if (v) atomicAdd(hist + t, v);
  }
}

// Block-wide exclusive scan of 256 values held by threads 0..255 (8 warps).
__device__ __forceinline__ uint32_t block_excl_scan256(uint32_t v, uint32_t* warp_tot) {
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  uint32_t inc = v;
#pragma unroll
  for (int off = 1; off < 32; off <<= 1) {
    uint32_t t = __shfl_up_sync(0xffffffffu, inc, off);
    if (lane >= off) inc += t;
  }
  if (lane == 31) warp_tot[w] = inc;
  __syncthreads();
  uint32_t add = 0;
  for (int k = 0; k < w; ++k) add += warp_tot[k];
  __syncthreads();
  return add + inc - v;
}

struct SortSmem {
  uint64_t keys[kSortTile];
  uint32_t vals[kSortTile];
  uint32_t wcnt[kSortThreads / 32][kRadix];  // per-warp digit counts -> offsets
  uint32_t digit_start[kRadix];              // tile-local exclusive digit offsets
  uint32_t gbase[kRadix];                    // global position of the tile's digit run
  uint32_t warp_tot[8];
  uint32_t tile;
};

// Resident CTAs per SM requested from the register allocator (A/B builds).
#ifndef SPH_SORT_MINB
#define SPH_SORT_MINB 4  // 4 x 256 threads: <= 64 registers, no spills (3 -> 4 CTAs per SM)
#endif
template <bool kFirst>
__global__ void __launch_bounds__(kSortThreads, SPH_SORT_MINB) onesweep_kernel(
    const uint64_t* __restrict__ kin, const uint32_t* __restrict__ vin, uint64_t* __restrict__ kout,
    uint32_t* __restrict__ vout, int64_t n, int shift, const uint32_t* __restrict__ hist,
    uint32_t* __restrict__ status, uint32_t* __restrict__ tile_ctr) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  SortSmem& S = *reinterpret_cast<SortSmem*>(smem_raw);
  const int tid = threadIdx.x, lane = tid & 31, w = tid >> 5;

  if (tid == 0) S.tile = atomicAdd(tile_ctr, 1u);
  for (int t = tid; t < (kSortThreads / 32) * kRadix; t += kSortThreads) (&S.wcnt[0][0])[t] = 0;
  __syncthreads();
  const uint32_t tile = S.tile;
  const int64_t base = (int64_t)tile * kSortTile;
  const int64_t seg = base + (int64_t)w * 32 * kSortKPT;

  uint64_t k[kSortKPT];
  uint32_t v[kSortKPT];
  uint32_t rank[kSortKPT];
#pragma unroll
  for (int j = 0; j < kSortKPT; ++j) {
    int64_t idx = seg + j * 32 + lane;
    bool valid = idx < n;
    k[j] = valid ? kin[idx] : ~0ull;
    v[j] = kFirst ? (uint32_t)idx : (valid ? vin[idx] : 0u);
  }
  // Stable rank within the warp's segment: vectors in order j, lanes in order.
#pragma unroll
  for (int j = 0; j < kSortKPT; ++j) {
    bool valid = seg + j * 32 + lane < n;
    uint32_t d = valid ? (uint32_t)((k[j] >> shift) & (kRadix - 1)) : 0x100u;
    uint32_t peers = __match_any_sync(0xffffffffu, d);
    uint32_t lt = __popc(peers & lanemask_lt());
    uint32_t cnt = valid ? S.wcnt[w][d] : 0u;
    rank[j] = cnt + lt;
    __syncwarp();
    if (valid && lt == 0) S.wcnt[w][d] = cnt + __popc(peers);
    __syncwarp();
  }
  __syncthreads();

  // Per digit: exclusive offsets over warps, tile total.
  uint32_t tile_cnt = 0;
  if (tid < kRadix) {
#pragma unroll
    for (int ww = 0; ww < kSortThreads / 32; ++ww) {
      uint32_t t = S.wcnt[ww][tid];
      S.wcnt[ww][tid] = tile_cnt;
      tile_cnt += t;
    }
    // Publish the aggregate (tile 0 publishes its inclusive prefix directly).
    st_relaxed(status + (size_t)tile * kRadix + tid, (tile == 0 ? kFlagInc : kFlagAgg) | tile_cnt);
  }
  // Tile-local digit starts and the pass's global digit starts (both scans by
  // threads 0..255; kSortThreads == kRadix).
  uint32_t dstart = block_excl_scan256(tid < kRadix ? tile_cnt : 0u, S.warp_tot);
  uint32_t gstart = block_excl_scan256(tid < kRadix ? hist[tid] : 0u, S.warp_tot);
  if (tid < kRadix) {
    uint32_t excl = 0;
    if (tile > 0) {
      int64_t j = (int64_t)tile - 1;
      while (true) {
        uint32_t s = ld_relaxed(status + (size_t)j * kRadix + tid);
        uint32_t flag = s & ~kValMask;
        if (flag == 0) continue;  // predecessor has not published yet
        excl += s & kValMask;
        if (flag == kFlagInc) break;
        --j;
      }
      st_relaxed(status + (size_t)tile * kRadix + tid, kFlagInc | (excl + tile_cnt));
    }
    S.digit_start[tid] = dstart;
    S.gbase[tid] = gstart + excl;
  }
  __syncthreads();

  // Reorder the tile in shared memory by (digit, stable rank).
#pragma unroll
  for (int j = 0; j < kSortKPT; ++j) {
    if (seg + j * 32 + lane < n) {
      uint32_t d = (uint32_t)((k[j] >> shift) & (kRadix - 1));
      uint32_t pos = S.digit_start[d] + S.wcnt[w][d] + rank[j];
      S.keys[pos] = k[j];
      S.vals[pos] = v[j];
    }
  }
  __syncthreads();
  const int cnt_valid = (int)std::min<int64_t>(kSortTile, n - base);
  for (int t = tid; t < cnt_valid; t += kSortThreads) {
    uint64_t key = S.keys[t];
    uint32_t d = (uint32_t)((key >> shift) & (kRadix - 1));
    uint32_t out = S.gbase[d] + (uint32_t)t - S.digit_start[d];
    kout[out] = key;
    vout[out] = S.vals[t];
  }
}

void sort_workspace(int64_t cap, size_t* hist_bytes, size_t* status_bytes) {
  int64_t tiles = std::max<int64_t>(1, div_up(cap, kSortTile));
  *hist_bytes = sizeof(uint32_t) * (kSortPasses * kRadix + kSortPasses);  // + tile counters
  *status_bytes = sizeof(uint32_t) * (size_t)tiles * kRadix * kSortPasses;
}

// Sorts F.n keys from key_in.  Returns the sorted keys and the permutation
// (perm[k] = input index of the k-th smallest) in *key_out / *perm_out, which
// point into the ping-pong buffers.
// Runs of keys equal in the sorted digits: after LSD passes over the digits
// skip..7 only, the order is sorted by key >> 8 skip, and equal prefixes keep
// the input order (stable passes).  Sorting every such run by the full key with
// a stable insertion sort then gives exactly the stable sort by the full key
// (ties keep the input order).  The keys arrive from last step's order with
// particles far apart compared with a level-10 cell, so the runs are almost all
// of length 1: the fixup is one read of the keys.  The longest run is recorded
// (DevScalars::sort_maxrun) and the host falls back to all 8 passes when runs
// grow long (launch_sort's `skip`, api.cu).
__global__ void __launch_bounds__(256) sort_fixup_kernel(uint64_t* __restrict__ key, uint32_t* __restrict__ val,
                                                         int64_t n, int shift, DevScalars* ds) {
  const int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (i >= n) return;
  const uint64_t h = key[i] >> shift;
  if (i > 0 && (key[i - 1] >> shift) == h) return;           // not the first of its run
  if (i + 1 >= n || (key[i + 1] >> shift) != h) return;      // run of one: nothing to do
  int64_t e = i + 2;
  while (e < n && (key[e] >> shift) == h) ++e;
  for (int64_t a = i + 1; a < e; ++a) {  // stable insertion sort of [i, e) by the full key
    const uint64_t k = key[a];
    const uint32_t v = val[a];
    int64_t b = a - 1;
    while (b >= i && key[b] > k) {
      key[b + 1] = key[b];
      val[b + 1] = val[b];
      --b;
    }
    key[b + 1] = k;
    val[b + 1] = v;
  }
  const unsigned long long len = (unsigned long long)(e - i);
  atomicMax(&ds->sort_maxrun, len);
}

cudaError_t launch_sort(const Fields& F, uint64_t* key_in, uint64_t* key_tmp, uint32_t* val_a,
                        uint32_t* val_b, uint32_t* hist, uint32_t* status, size_t status_bytes,
                        uint32_t** perm_out, uint64_t** key_out, cudaStream_t st, int skip) {
  const int64_t n = F.n;
  *perm_out = val_a;
  *key_out = key_in;
  if (n == 0) return cudaSuccess;
  const size_t smem = sizeof(SortSmem);
  cudaFuncSetAttribute(onesweep_kernel<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  cudaFuncSetAttribute(onesweep_kernel<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  cudaMemsetAsync(hist, 0, sizeof(uint32_t) * (kSortPasses * kRadix + kSortPasses), st);
  const int64_t tiles = div_up(n, kSortTile);
  cudaMemsetAsync(status, 0, sizeof(uint32_t) * (size_t)tiles * kRadix * kSortPasses, st);
  (void)status_bytes;
  // Few CTAs: every CTA ends with one global atomic per nonzero bin (8 x 256),
  // and with keys spread over the whole array every bin is nonzero, so the
  // flush contends on 2048 L2 addresses: 2 CTAs per SM keep it ~0.6M atomics.
  static int sms = 0;
  if (!sms) {
    int dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    sms = std::max(sms, 1);
  }
  int hb = (int)std::min<int64_t>(div_up(div_up(n, 8), kHistThreads), 2 * sms);
  sort_hist_kernel<<<hb, kHistThreads, 0, st>>>(key_in, n, hist); note_launch();
  uint32_t* tile_ctr = hist + kSortPasses * kRadix;
  uint64_t* ks[2] = {key_in, key_tmp};
  uint32_t* vs[2] = {val_a, val_b};
  int cur = 0;
  skip = std::max(0, std::min(skip, kSortPasses - 1));
  for (int p = skip; p < kSortPasses; ++p) {
    uint32_t* stp = status + (size_t)p * tiles * kRadix;
    if (p == skip)
      onesweep_kernel<true><<<(unsigned)tiles, kSortThreads, smem, st>>>(
          ks[cur], nullptr, ks[cur ^ 1], vs[cur ^ 1], n, p * kRadixBits, hist + p * kRadix, stp,
          tile_ctr + p);
    else
      onesweep_kernel<false><<<(unsigned)tiles, kSortThreads, smem, st>>>(
          ks[cur], vs[cur], ks[cur ^ 1], vs[cur ^ 1], n, p * kRadixBits, hist + p * kRadix, stp,
          tile_ctr + p);
    note_launch();
    cur ^= 1;
  }
  *key_out = ks[cur];
  *perm_out = vs[cur];
  if (skip > 0) {
    sort_fixup_kernel<<<(unsigned)div_up(n, 256), 256, 0, st>>>(ks[cur], vs[cur], n, skip * kRadixBits, F.ds);
    note_launch();
  }
  return cudaGetLastError();
}

// Gathers every persistent field into key order, dst_f[k] = src_f[perm[k]], and
// writes the two records the next phases gather from: the fp32 prefilter
// position pos4 = (x, y, z) - box_min and rec_d = {x, y, z, m} (density).
// HBM-bound: 11 x 8 B read (gather, near-identity permutation) + 11 x 8 B + 16 B
// + 32 B written per particle.
struct PermPtrs {
  const double* src[kNumStateF];
};

__global__ void __launch_bounds__(256) permute_kernel(Fields F, const uint32_t* __restrict__ perm,
                                                      PermPtrs P, const int64_t* __restrict__ id_src) {
  int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (i >= F.n) return;
  uint32_t p = perm[i];
  double v[kNumStateF];
#pragma unroll
  for (int f = 0; f < kNumStateF; ++f) {
    v[f] = __ldg(P.src[f] + p);
    F.f[f][i] = v[f];
  }
  F.id[i] = __ldg(id_src + p);
  const DevScalars* ds = F.ds;
  // w = 1 marks a ghost (the neighbour search flags the targets that touch one)
  F.pos4[i] = make_float4((float)(v[FX] - ds->box_min[0]), (float)(v[FY] - ds->box_min[1]),
                          (float)(v[FZ] - ds->box_min[2]), (__ldg(id_src + p) & SPH_GHOST_BIT) ? 1.f : 0.f);
  st4(F.rec_d + i, v[FX], v[FY], v[FZ], v[FM]);
}

void launch_permute(const Fields& Fdst, const uint32_t* perm, double* const* src,
                    const int64_t* id_src, cudaStream_t st) {
  if (Fdst.n == 0) return;
  PermPtrs P;
  for (int f = 0; f < kNumStateF; ++f) P.src[f] = src[f];
  permute_kernel<<<(unsigned)div_up(Fdst.n, 256), 256, 0, st>>>(Fdst, perm, P, id_src);
  note_launch();
}

}  // namespace sph
