// k_gravity.cu -- phase GRAVITY: self-gravity by a Barnes-Hut octree with
// quadrupole moments on the Morton cells (the Evrard collapse
// workload of P:108; definitions in include/sph.h, reading 20).
//
// The tree is the Morton grid itself: the particles are already sorted by key,
// so a cell at level l is the key prefix key >> 3(21-l) and its particles are a
// contiguous range.  Dense levels 0..Lt (Lt = cfg.grav_level):
//  1. grav_cells_kernel   leaf ranges at level Lt (like the neighbour grid);
//  2. grav_leaf_kernel    per leaf: mass, centre of mass, traceless quadrupole
//                         Q_ab = sum m (3 d_a d_b - d^2 delta_ab) about the COM;
//  3. grav_up_kernel      per level, parents from their 8 children (parallel-axis
//                         shift of each child's quadrupole to the parent's COM);
//  4. grav_walk_kernel    one warp per 32 consecutive (Morton-adjacent) targets
//                         walks the tree depth first with a shared-memory stack:
//                         a cell is accepted as a multipole when side < theta *
//                         distance(target box, COM) (one warp-uniform decision for
//                         the 32 targets, no divergence), opened otherwise; leaves
//                         that are not accepted are summed directly with the
//                         Plummer-softened pair force.  Children are pushed in
//                         reverse so leaves are visited in ascending particle
//                         order: with theta = 0 the walk is the direct sum of the
//                         oracle, in the oracle's order.
// Bound: FP64 (direct pairs ~20 DP ops, multipoles ~45); the moments are
// HBM-light (96 B per cell).
#include <algorithm>

#include "sph_internal.cuh"

namespace sph {

__host__ __device__ inline int64_t grav_level_off(int l) { return ((int64_t(1) << (3 * l)) - 1) / 7; }

__global__ void __launch_bounds__(256) grav_cells_kernel(int64_t n, const uint64_t* __restrict__ key, int Lt,
                                                         uint32_t* __restrict__ cs) {
  const int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (i >= n) return;
  const int shift = 3 * (21 - Lt);
  const int64_t ncell = int64_t(1) << (3 * Lt);
  const int64_t ck = (int64_t)(key[i] >> shift);
  const int64_t prev = i > 0 ? (int64_t)(key[i - 1] >> shift) : -1;
  for (int64_t c = prev + 1; c <= ck; ++c) cs[c] = (uint32_t)i;
  if (i == n - 1)
    for (int64_t c = ck + 1; c <= ncell; ++c) cs[c] = (uint32_t)n;
}

__device__ __forceinline__ void store_mom(Rec4* g, int64_t cell, double m, const double c[3], const double q[6]) {
  st4(g + 3 * cell + 0, m, c[0], c[1], c[2]);
  st4(g + 3 * cell + 1, q[0], q[1], q[2], q[3]);
  st4(g + 3 * cell + 2, q[4], q[5], 0.0, 0.0);
}

__global__ void __launch_bounds__(256) grav_leaf_kernel(Fields F, int Lt) {
  const int64_t c = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (c >= (int64_t(1) << (3 * Lt))) return;
  const uint32_t s = F.gcell_start[c], e = F.gcell_start[c + 1];
  double m = 0, com[3] = {0, 0, 0}, q[6] = {0, 0, 0, 0, 0, 0};
  for (uint32_t j = s; j < e; ++j) {
    const Rec4 r = ldg4(F.rec_d + j);
    m += r.d;
    com[0] = fma(r.d, r.a, com[0]);
    com[1] = fma(r.d, r.b, com[1]);
    com[2] = fma(r.d, r.c, com[2]);
  }
  if (m > 0) {
    for (int a = 0; a < 3; ++a) com[a] /= m;
    for (uint32_t j = s; j < e; ++j) {
      const Rec4 r = ldg4(F.rec_d + j);
      const double d[3] = {r.a - com[0], r.b - com[1], r.c - com[2]};
      const double d2 = d[0] * d[0] + d[1] * d[1] + d[2] * d[2];
      q[0] += r.d * (3 * d[0] * d[0] - d2);
      q[1] += r.d * (3 * d[0] * d[1]);
      q[2] += r.d * (3 * d[0] * d[2]);
      q[3] += r.d * (3 * d[1] * d[1] - d2);
      q[4] += r.d * (3 * d[1] * d[2]);
      q[5] += r.d * (3 * d[2] * d[2] - d2);
    }
  }
  store_mom(F.gmom, grav_level_off(Lt) + c, m, com, q);
}

__global__ void __launch_bounds__(256) grav_up_kernel(Fields F, int l) {
  const int64_t c = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (c >= (int64_t(1) << (3 * l))) return;
  const int64_t ch0 = grav_level_off(l + 1) + 8 * c;
  double m = 0, com[3] = {0, 0, 0}, q[6] = {0, 0, 0, 0, 0, 0};
  Rec4 k0[8];
#pragma unroll
  for (int k = 0; k < 8; ++k) {
    k0[k] = ldg4(F.gmom + 3 * (ch0 + k));
    m += k0[k].a;
    com[0] = fma(k0[k].a, k0[k].b, com[0]);
    com[1] = fma(k0[k].a, k0[k].c, com[1]);
    com[2] = fma(k0[k].a, k0[k].d, com[2]);
  }
  if (m > 0) {
    for (int a = 0; a < 3; ++a) com[a] /= m;
#pragma unroll
    for (int k = 0; k < 8; ++k) {
      if (k0[k].a == 0.0) continue;
      const Rec4 k1 = ldg4(F.gmom + 3 * (ch0 + k) + 1), k2 = ldg4(F.gmom + 3 * (ch0 + k) + 2);
      const double d[3] = {k0[k].b - com[0], k0[k].c - com[1], k0[k].d - com[2]};
      const double d2 = d[0] * d[0] + d[1] * d[1] + d[2] * d[2], mk = k0[k].a;
      q[0] += k1.a + mk * (3 * d[0] * d[0] - d2);
      q[1] += k1.b + mk * (3 * d[0] * d[1]);
      q[2] += k1.c + mk * (3 * d[0] * d[2]);
      q[3] += k1.d + mk * (3 * d[1] * d[1] - d2);
      q[4] += k2.a + mk * (3 * d[1] * d[2]);
      q[5] += k2.b + mk * (3 * d[2] * d[2] - d2);
    }
  }
  store_mom(F.gmom, grav_level_off(l) + c, m, com, q);
}

constexpr int kGravThreads = 128;
constexpr int kGravWarps = kGravThreads / 32;
#ifndef SPH_GRAV_SPEC
#define SPH_GRAV_SPEC 1  // a child's three moment chunks loaded together
#endif
constexpr int kGravPop = 4;     // stack nodes examined per round (8 children each)
constexpr int kGravStack = 256;
// per level at most 32 - kGravPop children wait below the top round's 32
static_assert(kGravStack >= 8 * (32 - kGravPop) + 32, "stack for leaf levels <= 8");

struct GravSmem {
  uint32_t stack[kGravStack];   // parents whose 8 children are still to examine
  double mom[32][10];           // the accepted children's moments (m, com, Q)
  double px[32], py[32], pz[32], pm[32];  // a batch of leaf particles
  uint32_t pj[32];              // their particle indices (the self pair)
  // fp32 terms (GravParams::fp32): moments with the COM relative to the group's
  // centre, and leaf particles relative to it
  // fp32 terms: the accepted children's m, com - o (3), Q (6), compacted in
  // rank order and interleaved by pairs: momp[r / 2][field][r % 2] (one
  // 64-bit load = a field of two cells)
  float momp[16][10][2];
  float pxf[32], pyf[32], pzf[32], pmf[32];
};

// Multipole (monopole + traceless quadrupole, unsoftened) of cell moments q at
// target offset r = x_i - com.
__device__ __forceinline__ void add_multipole(const double* q, double xi, double yi, double zi, double Gc,
                                              double& ax, double& ay, double& az, double& phi) {
  const double rx = xi - q[1], ry = yi - q[2], rz = zi - q[3];
  const double r2 = rx * rx + ry * ry + rz * rz;
  const double ir = rsqrt(r2), ir2 = ir * ir, ir3 = ir * ir2, ir5 = ir3 * ir2;
  const double Qx = q[4] * rx + q[5] * ry + q[6] * rz;
  const double Qy = q[5] * rx + q[7] * ry + q[8] * rz;
  const double Qz = q[6] * rx + q[8] * ry + q[9] * rz;
  const double rQr = rx * Qx + ry * Qy + rz * Qz;
  const double mono = -Gc * q[0] * ir3;
  const double quad = -2.5 * Gc * rQr * ir5 * ir2;
  ax += mono * rx + Gc * Qx * ir5 + quad * rx;
  ay += mono * ry + Gc * Qy * ir5 + quad * ry;
  az += mono * rz + Gc * Qz * ir5 + quad * rz;
  phi += -Gc * q[0] * ir - 0.5 * Gc * rQr * ir5;
}

// The same multipole with fp32 terms: r = (x_i - o) - (com - o), both rounded
// to fp32 relative to the group's centre o (|x_i - o| is within the group and
// |com - o| <= |r| + the group's size, so the rounding of r is ~1e-7 of |r|).
__device__ __forceinline__ void add_multipole_f(const float* q, float xf, float yf, float zf, float Gc,
                                                float& ax, float& ay, float& az, float& phi) {
  const float rx = xf - q[1], ry = yf - q[2], rz = zf - q[3];
  const float r2 = fmaf(rx, rx, fmaf(ry, ry, rz * rz));
  const float ir = rsqrtf(r2), ir2 = ir * ir, ir3 = ir * ir2, ir5 = ir3 * ir2;
  const float Qx = fmaf(q[4], rx, fmaf(q[5], ry, q[6] * rz));
  const float Qy = fmaf(q[5], rx, fmaf(q[7], ry, q[8] * rz));
  const float Qz = fmaf(q[6], rx, fmaf(q[8], ry, q[9] * rz));
  const float rQr = fmaf(rx, Qx, fmaf(ry, Qy, rz * Qz));
  const float gi5 = Gc * ir5;
  const float s = -Gc * q[0] * ir3 - 2.5f * rQr * gi5 * ir2;  // mono + quad (radial)
  ax = fmaf(s, rx, fmaf(gi5, Qx, ax));
  ay = fmaf(s, ry, fmaf(gi5, Qy, ay));
  az = fmaf(s, rz, fmaf(gi5, Qz, az));
  phi -= fmaf(0.5f * rQr, gi5, Gc * q[0] * ir);
}

// Two multipoles per instruction (packed f32x2, FFMA2 / FMUL2): q2 holds the
// fields of cells a (low half) and b (high half); the sums go to packed
// accumulators (low: a's, high: b's).  Same operations as add_multipole_f.
__device__ __forceinline__ void add_multipole_f2(const float (*q2)[2], unsigned long long xf2,
                                                 unsigned long long yf2, unsigned long long zf2,
                                                 unsigned long long G2, unsigned long long& ax,
                                                 unsigned long long& ay, unsigned long long& az,
                                                 unsigned long long& phi) {
  auto ld = [&](int k) { return *reinterpret_cast<const unsigned long long*>(q2[k]); };
  const unsigned long long m = ld(0);
  const unsigned long long rx = sub2(xf2, ld(1)), ry = sub2(yf2, ld(2)), rz = sub2(zf2, ld(3));
  const unsigned long long r2 = fma2(rx, rx, fma2(ry, ry, mul2(rz, rz)));
  float r2a, r2b;
  unpack2(r2, r2a, r2b);
  const unsigned long long ir = pack2(rsqrtf(r2a), rsqrtf(r2b));
  const unsigned long long ir2 = mul2(ir, ir), ir3 = mul2(ir, ir2), ir5 = mul2(ir3, ir2);
  const unsigned long long q4 = ld(4), q5 = ld(5), q6 = ld(6), q7 = ld(7), q8 = ld(8), q9 = ld(9);
  const unsigned long long Qx = fma2(q4, rx, fma2(q5, ry, mul2(q6, rz)));
  const unsigned long long Qy = fma2(q5, rx, fma2(q7, ry, mul2(q8, rz)));
  const unsigned long long Qz = fma2(q6, rx, fma2(q8, ry, mul2(q9, rz)));
  const unsigned long long rQr = fma2(rx, Qx, fma2(ry, Qy, mul2(rz, Qz)));
  const unsigned long long gi5 = mul2(G2, ir5);
  const unsigned long long Gm = mul2(G2, m);
  // s = -G m ir3 - 2.5 rQr gi5 ir2
  const unsigned long long s = fma2(mul2(splat2(-2.5f), rQr), mul2(gi5, ir2), mul2(splat2(-1.f), mul2(Gm, ir3)));
  ax = fma2(s, rx, fma2(gi5, Qx, ax));
  ay = fma2(s, ry, fma2(gi5, Qy, ay));
  az = fma2(s, rz, fma2(gi5, Qz, az));
  // phi -= 0.5 rQr gi5 + G m ir
  phi = sub2(phi, fma2(mul2(splat2(0.5f), rQr), gi5, mul2(Gm, ir)));
}

// One warp per 32 consecutive targets.  The stack holds parents; popping one
// examines its 8 children together (lanes 0-7 load and classify one child each:
// one memory round trip per 8 cells instead of 8 dependent ones): accepted
// children are evaluated as multipoles from shared memory, leaf children are
// summed directly in batches of 32 particles staged in shared memory (one load
// per lane), the other children are pushed (in reverse: ascending pop order).
// With theta = 0 every child of a level-(Lt-1) node is a leaf and no other node
// has leaf children, so the direct sums run over ascending particle indices.
// One walk for the lanes in `mine` (a group of the tile's targets): the
// opening test uses the bounding box of the group's targets only; the other
// lanes follow the warp-uniform walk and discard what they compute.
template <bool kF32>
__device__ __forceinline__ void walk_group(const Fields& F, const GravParams& G, GravSmem& S, int lane,
                                           int64_t i, bool active, bool mine, double& tax, double& tay,
                                           double& taz, double& tphi) {
  const int64_t ii = active ? i : F.n - 1;
  const double xi = F.f[FX][ii], yi = F.f[FY][ii], zi = F.f[FZ][ii];
  double lo[3] = {mine ? xi : INFINITY, mine ? yi : INFINITY, mine ? zi : INFINITY};
  double hi[3] = {mine ? xi : -INFINITY, mine ? yi : -INFINITY, mine ? zi : -INFINITY};
#pragma unroll
  for (int a = 0; a < 3; ++a)
#pragma unroll
    for (int off = 16; off > 0; off >>= 1) {
      lo[a] = fmin(lo[a], __shfl_xor_sync(0xffffffffu, lo[a], off));
      hi[a] = fmax(hi[a], __shfl_xor_sync(0xffffffffu, hi[a], off));
    }
  const DevScalars* ds = F.ds;
  const double Lmax = fmax(ds->box_max[0] - ds->box_min[0],
                           fmax(ds->box_max[1] - ds->box_min[1], ds->box_max[2] - ds->box_min[2]));
  const double th2 = G.theta * G.theta, eps2 = G.eps * G.eps, Gc = G.G;
  const int Lt = G.level;
  double ax = 0, ay = 0, az = 0, phi = 0;
  unsigned long long n_mp = 0, n_pp = 0, n_pop = 0;  // diagnostics (warp-uniform)
  // fp32 terms: positions relative to the group's centre o (warp-uniform)
  const double ox = 0.5 * (lo[0] + hi[0]), oy = 0.5 * (lo[1] + hi[1]), oz = 0.5 * (lo[2] + hi[2]);
  const float xf = (float)(xi - ox), yf = (float)(yi - oy), zf = (float)(zi - oz);
  const float Gf = (float)Gc, eps2f = (float)eps2;
  const unsigned long long xf2 = splat2(xf), yf2 = splat2(yf), zf2 = splat2(zf), G2 = splat2(Gf);

  // the root itself: accepted, a leaf (Lt = 0 is not allowed) or opened
  int sp = 0;
  {
    const Rec4 m0 = ldg4(F.gmom);
    if (m0.a == 0.0) goto done;
    double dd2 = 0;
    const double cc[3] = {m0.b, m0.c, m0.d};
#pragma unroll
    for (int a = 0; a < 3; ++a) {
      const double t = fmax(fmax(lo[a] - cc[a], cc[a] - hi[a]), 0.0);
      dd2 += t * t;
    }
    if (Lmax * Lmax < th2 * dd2) {
      const Rec4 m1 = ldg4(F.gmom + 1), m2 = ldg4(F.gmom + 2);
      const double q[10] = {m0.a, m0.b, m0.c, m0.d, m1.a, m1.b, m1.c, m1.d, m2.a, m2.b};
      add_multipole(q, xi, yi, zi, Gc, ax, ay, az, phi);
      goto done;
    }
    if (lane == 0) S.stack[0] = 0u;  // open the root
    sp = 1;
    __syncwarp();
  }
  while (sp > 0) {
    // up to kGravPop nodes from the top of the stack (the smallest first) are
    // examined together: lane 8g + k takes child k of popped node g (one
    // memory round trip for up to 32 cells).  With theta = 0 the order of the
    // direct sums is unchanged: the popped nodes are ascending and no smaller
    // popped node is shallower than a larger one, so leaves still come in
    // ascending particle order.
    const int np = min(sp, kGravPop);
    const int gq = lane >> 3, kq = lane & 7;
    const uint32_t e = gq < np ? S.stack[sp - 1 - gq] : 0u;
    __syncwarp();
    sp -= np;
    n_pop += np;
    bool acc = false, open = false, leaf = false;
    int l = 0;
    uint32_t cl = 0;  // the child's index at level l
    uint32_t leaf_s = 0, leaf_n = 0;  // a leaf child's particle range
    float qf[10];                     // an accepted child's moments (fp32 terms)
    if (gq < np) {
      l = (int)(e >> 28) + 1;
      cl = 8u * (e & 0x0fffffffu) + (uint32_t)kq;
      const int64_t gc = grav_level_off(l) + cl;
      // the whole record in one round trip (m1, m2 are needed if accepted)
      const Rec4 m0 = ldg4(F.gmom + 3 * gc);
      Rec4 m1, m2;
      if (SPH_GRAV_SPEC) {
        m1 = ldg4(F.gmom + 3 * gc + 1);
        m2 = ldg4(F.gmom + 3 * gc + 2);
      }
      if (m0.a != 0.0) {
        const double side = Lmax / (double)(1 << l);
        double dd2 = 0;
        const double cc[3] = {m0.b, m0.c, m0.d};
#pragma unroll
        for (int a = 0; a < 3; ++a) {
          const double t = fmax(fmax(lo[a] - cc[a], cc[a] - hi[a]), 0.0);
          dd2 += t * t;
        }
        if (side * side < th2 * dd2) {
          acc = true;
          if (!SPH_GRAV_SPEC) {
            m1 = ldg4(F.gmom + 3 * gc + 1);
            m2 = ldg4(F.gmom + 3 * gc + 2);
          }
          if (kF32) {
            qf[0] = (float)m0.a;
            qf[1] = (float)(m0.b - ox); qf[2] = (float)(m0.c - oy); qf[3] = (float)(m0.d - oz);
            qf[4] = (float)m1.a; qf[5] = (float)m1.b; qf[6] = (float)m1.c; qf[7] = (float)m1.d;
            qf[8] = (float)m2.a; qf[9] = (float)m2.b;
          } else {
            double* q = S.mom[lane];
            q[0] = m0.a; q[1] = m0.b; q[2] = m0.c; q[3] = m0.d;
            q[4] = m1.a; q[5] = m1.b; q[6] = m1.c; q[7] = m1.d; q[8] = m2.a; q[9] = m2.b;
          }
        } else if (l == Lt) {
          leaf = true;
          leaf_s = F.gcell_start[cl];
          leaf_n = F.gcell_start[cl + 1] - leaf_s;
        } else {
          open = true;
        }
      }
    }
    const uint32_t am = __ballot_sync(0xffffffffu, acc);
    const uint32_t lm = __ballot_sync(0xffffffffu, leaf);
    const uint32_t om = __ballot_sync(0xffffffffu, open);
    if (kF32 && acc) {
      const int r = __popc(am & ((1u << lane) - 1u));  // rank among the accepted
#pragma unroll
      for (int f = 0; f < 10; ++f) S.momp[r >> 1][f][r & 1] = qf[f];
    }
    __syncwarp();
    // multipoles, two at a time into separate accumulators (independent
    // dependency chains: the rsqrt + quadrupole chain is latency-bound)
    n_mp += __popc(am);
    if (kF32) {
      // this round's multipole terms, two cells per packed instruction, summed
      // in fp32, then added in fp64 (an odd last cell pairs with a zero-mass,
      // zero-Q slot: its terms are exactly 0)
      const int na = __popc(am);
      if (na & 1) {
        // far away (r^2 ~ 1e36 stays finite), no mass, no Q: every term is 0
        if (lane < 10) S.momp[na >> 1][lane][1] = lane >= 1 && lane <= 3 ? 1e18f : 0.f;
        __syncwarp();
      }
      unsigned long long fx = 0ull, fy = 0ull, fz = 0ull, fphi = 0ull;
      for (int r = 0; r < na; r += 2)
        add_multipole_f2(S.momp[r >> 1], xf2, yf2, zf2, G2, fx, fy, fz, fphi);
      float a0, a1;
      unpack2(fx, a0, a1);
      ax += (double)a0 + (double)a1;
      unpack2(fy, a0, a1);
      ay += (double)a0 + (double)a1;
      unpack2(fz, a0, a1);
      az += (double)a0 + (double)a1;
      unpack2(fphi, a0, a1);
      phi += (double)a0 + (double)a1;
    } else {
      double bx = 0, by = 0, bz = 0, bphi = 0;
      uint32_t m = am;
      for (; __popc(m) >= 2; m &= m - 1, m &= m - 1) {
        const int k0 = __ffs(m) - 1;
        const int k1 = __ffs(m & (m - 1)) - 1;
        add_multipole(S.mom[k0], xi, yi, zi, Gc, ax, ay, az, phi);
        add_multipole(S.mom[k1], xi, yi, zi, Gc, bx, by, bz, bphi);
      }
      if (m) add_multipole(S.mom[__ffs(m) - 1], xi, yi, zi, Gc, ax, ay, az, phi);
      ax += bx;
      ay += by;
      az += bz;
      phi += bphi;
    }
    // leaves.  When the round's leaves hold <= 32 particles together (small
    // leaves: the common case at the default level), their particles are
    // concatenated in ascending lane (= cell) order and staged as one batch;
    // otherwise each leaf is streamed in batches of 32 of its own.
    uint32_t ltotal = 0, loff = 0;
    if (lm) {
      loff = leaf_n;  // inclusive prefix over lanes of the leaf sizes
#pragma unroll
      for (int d = 1; d < 32; d <<= 1) {
        const uint32_t v = __shfl_up_sync(0xffffffffu, loff, d);
        if (lane >= d) loff += v;
      }
      ltotal = __shfl_sync(0xffffffffu, loff, 31);
      loff -= leaf_n;  // exclusive
    }
    if (lm && ltotal <= 32u) {
      const uint32_t total = ltotal, off = loff;
      n_pp += total;
      for (uint32_t b0 = 0; b0 < total; b0 += 32) {
        const uint32_t nb = min(32u, total - b0);
        const uint32_t g = b0 + (uint32_t)lane;
        // owner leaf of item g: the leaf lanes are few; each claims its items
        uint32_t j = 0;
        for (uint32_t m = lm; m; m &= m - 1) {
          const int q = __ffs(m) - 1;
          const uint32_t oq = __shfl_sync(0xffffffffu, off, q), nq = __shfl_sync(0xffffffffu, leaf_n, q),
                         sq = __shfl_sync(0xffffffffu, leaf_s, q);
          if (g - oq < nq) j = sq + (g - oq);
        }
        __syncwarp();
        if (g < total) {
          const Rec4 r = ldg4(F.rec_d + j);
          S.pj[lane] = j;
          if (kF32) {
            S.pxf[lane] = (float)(r.a - ox);
            S.pyf[lane] = (float)(r.b - oy);
            S.pzf[lane] = (float)(r.c - oz);
            S.pmf[lane] = (float)r.d;
          } else {
            S.px[lane] = r.a;
            S.py[lane] = r.b;
            S.pz[lane] = r.c;
            S.pm[lane] = r.d;
          }
        }
        __syncwarp();
        // the self pair is skipped by a zero mass (branch-free, unrolled by 4
        // for independent rsqrt chains)
        if (kF32) {
          float fx = 0.f, fy = 0.f, fz = 0.f, fphi = 0.f;
#pragma unroll 4
          for (uint32_t t = 0; t < nb; ++t) {
            const bool me = (int64_t)S.pj[t] == ii;
            const float mt = me ? 0.f : S.pmf[t];
            const float dx = S.pxf[t] - xf, dy = S.pyf[t] - yf, dz = S.pzf[t] - zf;
            const float r2 = me ? 1.f : fmaf(dx, dx, fmaf(dy, dy, fmaf(dz, dz, eps2f)));
            const float ir = rsqrtf(r2);
            const float gm = Gf * mt * ir;
            const float s3 = gm * ir * ir;
            fx = fmaf(s3, dx, fx);
            fy = fmaf(s3, dy, fy);
            fz = fmaf(s3, dz, fz);
            fphi -= gm;
          }
          ax += fx;
          ay += fy;
          az += fz;
          phi += fphi;
        } else {
#pragma unroll 4
          for (uint32_t t = 0; t < nb; ++t) {
            const bool me = (int64_t)S.pj[t] == ii;
            const double mt = me ? 0.0 : S.pm[t];
            const double dx = S.px[t] - xi, dy = S.py[t] - yi, dz = S.pz[t] - zi;
            const double r2 = me ? 1.0 : dx * dx + dy * dy + dz * dz + eps2;  // finite with eps = 0
            const double ir = rsqrt(r2);
            const double gm = Gc * mt * ir;
            const double s3 = gm * ir * ir;
            ax = fma(s3, dx, ax);
            ay = fma(s3, dy, ay);
            az = fma(s3, dz, az);
            phi -= gm;
          }
        }
      }
    }
    // leaves, ascending: particles in batches of 32 through shared memory
    for (uint32_t m = ltotal > 32u ? lm : 0u; m; m &= m - 1) {
      const int q = __ffs(m) - 1;
      const uint32_t s = __shfl_sync(0xffffffffu, leaf_s, q), en = s + __shfl_sync(0xffffffffu, leaf_n, q);
      for (uint32_t b = s; b < en; b += 32) {
        const uint32_t nb = min(32u, en - b);
        n_pp += nb;
        __syncwarp();
        if ((uint32_t)lane < nb) {
          const Rec4 r = ldg4(F.rec_d + b + lane);
          if (kF32) {
            S.pxf[lane] = (float)(r.a - ox);
            S.pyf[lane] = (float)(r.b - oy);
            S.pzf[lane] = (float)(r.c - oz);
            S.pmf[lane] = (float)r.d;
          } else {
            S.px[lane] = r.a;
            S.py[lane] = r.b;
            S.pz[lane] = r.c;
            S.pm[lane] = r.d;
          }
        }
        __syncwarp();
        // the self pair is skipped by a zero mass (branch-free, unrolled by 4
        // for independent rsqrt chains)
        const int64_t self = ii - (int64_t)b;
        if (kF32) {
          float fx = 0.f, fy = 0.f, fz = 0.f, fphi = 0.f;
#pragma unroll 4
          for (uint32_t t = 0; t < nb; ++t) {
            const bool me = (int64_t)t == self;
            const float mt = me ? 0.f : S.pmf[t];
            const float dx = S.pxf[t] - xf, dy = S.pyf[t] - yf, dz = S.pzf[t] - zf;
            const float r2 = me ? 1.f : fmaf(dx, dx, fmaf(dy, dy, fmaf(dz, dz, eps2f)));
            const float ir = rsqrtf(r2);
            const float gm = Gf * mt * ir;
            const float s3 = gm * ir * ir;
            fx = fmaf(s3, dx, fx);
            fy = fmaf(s3, dy, fy);
            fz = fmaf(s3, dz, fz);
            fphi -= gm;
          }
          ax += fx;
          ay += fy;
          az += fz;
          phi += fphi;
        } else {
#pragma unroll 4
          for (uint32_t t = 0; t < nb; ++t) {
            const bool me = (int64_t)t == self;
            const double mt = me ? 0.0 : S.pm[t];
            const double dx = S.px[t] - xi, dy = S.py[t] - yi, dz = S.pz[t] - zi;
            const double r2 = me ? 1.0 : dx * dx + dy * dy + dz * dz + eps2;  // finite with eps = 0
            const double ir = rsqrt(r2);
            const double gm = Gc * mt * ir;
            const double s3 = gm * ir * ir;
            ax = fma(s3, dx, ax);
            ay = fma(s3, dy, ay);
            az = fma(s3, dz, az);
            phi -= gm;
          }
        }
      }
    }
    // opened children: pushed in reverse so they pop in ascending order
    const int no = __popc(om);
    if (open) {
      const int rank_from_top = __popc(om & ((1u << lane) - 1u));  // 0 for the lowest child
      S.stack[sp + no - 1 - rank_from_top] = ((uint32_t)l << 28) | cl;
    }
    sp += no;
    __syncwarp();
  }
done:
  if (lane == 0) {
    atomicAdd(&F.ds->grav_mp, n_mp);
    atomicAdd(&F.ds->grav_pp, n_pp);
    atomicAdd(&F.ds->grav_pops, n_pop);
  }
  if (mine) {
    tax += ax;
    tay += ay;
    taz += az;
    tphi += phi;
  }
  __syncwarp();  // the shared stack is reused by the next walk
}

// A tile of 32 Morton-consecutive targets is walked once per group of targets
// sharing a cell of side 4 leaf cells (level Lt - 2): a tile that straddles a
// jump of the Morton curve (e.g. across the empty corners of the box around
// an Evrard sphere) would otherwise get a box so large that nothing is
// accepted and its walk degenerates to the direct sum over all particles (one
// such tile took as long as all the others together).
__device__ __forceinline__ void walk_tile(const Fields& F, const GravParams& G, GravSmem& S, int lane,
                                          int64_t i) {
  const bool active = i < F.n;
  const int Lg = max(G.level - 2, 0);
  const unsigned long long ck =
      active ? (unsigned long long)(F.key[i] >> (3 * (21 - Lg))) : (0xffffffff00000000ull | (unsigned)lane);
  const uint32_t peers = __match_any_sync(0xffffffffu, ck);
  uint32_t leaders = __ballot_sync(0xffffffffu, active && (peers & ((1u << lane) - 1u)) == 0);
  double ax = 0, ay = 0, az = 0, phi = 0;
  while (leaders) {
    const int ld = __ffs(leaders) - 1;
    leaders &= leaders - 1;
    const uint32_t gm = __shfl_sync(0xffffffffu, peers, ld);
    if (G.fp32) walk_group<true>(F, G, S, lane, i, active, ((gm >> lane) & 1u) != 0, ax, ay, az, phi);
    else walk_group<false>(F, G, S, lane, i, active, ((gm >> lane) & 1u) != 0, ax, ay, az, phi);
  }
  if (active) {
    F.ax[i] += ax;
    F.ay[i] += ay;
    F.az[i] += az;
    F.phi[i] = phi;
  }
}

// Persistent grid; warps take 32-target tiles from an atomic counter.  The
// cost of a tile varies by an order of magnitude across an Evrard sphere (the
// centre is dense), so a static one-block-per-tile grid left the SMs idle
// half of the time waiting on the slow central blocks.
__global__ void __launch_bounds__(kGravThreads) grav_walk_kernel(Fields F, GravParams G) {
  __shared__ GravSmem s_w[kGravWarps];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int64_t ntiles = div_up(F.n, 32);
  while (true) {
    unsigned long long t = 0;
    if (lane == 0) t = atomicAdd(&F.ds->grav_next, 1ull);
    t = __shfl_sync(0xffffffffu, t, 0);
    if ((int64_t)t >= ntiles) break;
    walk_tile(F, G, s_w[warp], lane, (int64_t)t * 32 + lane);
  }
}

void launch_gravity(const Fields& F, const GravParams& G, cudaStream_t st) {
  if (F.n == 0) return;
  cudaMemsetAsync(&F.ds->grav_mp, 0, 4 * sizeof(unsigned long long), st);  // diagnostics + tile counter
  const int Lt = G.level;
  grav_cells_kernel<<<(unsigned)div_up(F.n, 256), 256, 0, st>>>(F.n, F.key, Lt, F.gcell_start);
  grav_leaf_kernel<<<(unsigned)div_up(int64_t(1) << (3 * Lt), 256), 256, 0, st>>>(F, Lt);
  note_launch(2);
  for (int l = Lt - 1; l >= 0; --l) {
    grav_up_kernel<<<(unsigned)div_up(int64_t(1) << (3 * l), 256), 256, 0, st>>>(F, l);
    note_launch();
  }
  static int resident = 0;  // SMs x resident CTAs of the walk
  if (!resident) {
    int dev = 0, sms = 0, per = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, grav_walk_kernel, kGravThreads, 0);
    resident = std::max(1, sms * std::max(per, 1));
  }
  const int64_t grid = std::min<int64_t>(div_up(F.n, kGravThreads), resident);
  grav_walk_kernel<<<(unsigned)grid, kGravThreads, 0, st>>>(F, G);
  note_launch();
}

}  // namespace sph
