// api.cu -- the C ABI of include/sph.h: arena sub-allocation, the stage machine,
// phase wrappers with CUDA-event timing, NVML energy accounting and the
// per-phase clock policy.  All compute is in the k_*.cu kernels.
#include <stdarg.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>

#include <algorithm>
#include <atomic>
#include <chrono>
#include <mutex>
#include <thread>
#include <vector>

#include "nvml_dyn.h"
#include "sph_internal.cuh"

using namespace sph;

std::atomic<long long> sph::g_launches{0};

namespace {

enum Stage { S_INIT = 0, S_PART, S_TREE, S_NBR, S_DENS, S_EOS, S_IAD, S_MOM, S_DT };

const char* kPhaseNames[SPH_NPHASES] = {"keys",    "sort",    "cells", "neighbors",
                                        "density", "eos",     "iad",   "momentum_energy",
                                        "timestep", "update",  "stir", "gravity",
                                        "gradh"};

thread_local char g_err[512] = "";

constexpr size_t kAlign = 256;
inline size_t align_up(size_t v) { return (v + kAlign - 1) / kAlign * kAlign; }

int level_cap_for(const sph_config* c) {
  int L = std::min(c->max_cell_level, 10);
  int64_t limit = std::max<int64_t>(8 * c->n_capacity, 512);
  while (L > 0 && (int64_t(1) << (3 * L)) > limit) --L;
  return std::max(L, 0);
}

#ifndef SPH_SORT_SKIP
#define SPH_SORT_SKIP 4  // A/B builds
#endif
constexpr int kSortSkipDefault = SPH_SORT_SKIP;  // LSD passes over digits 4..7 (the top 31 key bits)
constexpr unsigned long long kSortMaxRun = 64;

struct PhaseRow {
  int64_t calls = 0;
  double seconds = 0, joules = 0, mhz_sum = 0;
  int64_t mhz_n = 0;
  unsigned locked = 0;
  bool avail = false;
};

}  // namespace

struct sph_ctx {
  sph_config cfg;
  Params P;
  cudaStream_t st = nullptr;
  int64_t n = 0;
  int level_cap = 0;
  // arena slices
  double* state[2][kNumStateF];
  int64_t* ids[2];
  int cur = 0;
  uint64_t *keyA, *keyB, *key_sorted;
  uint32_t *valA, *valB;
  double *rho, *p, *c, *vol, *prho2, *wq, *wk, *C[6], *ax, *ay, *az, *du;
  double *divv, *curl[3], *bal;
  Rec4* rec_iv = nullptr;
  double* phi = nullptr;
  double* omega = nullptr;  // cfg.gradh
  double* vsig = nullptr;   // cfg.dt_vsig
  bool gradh_done = false;  // GRADH ran since the last EOS (cfg.gradh)
  uint32_t* gcell_start = nullptr;
  Rec4* gmom = nullptr;
  int32_t *nc, *nbr, *nrows;
  uint32_t* cell_start;
  float4* pos4;
  Rec4 *rec_d, *rec_i, *rec_m;
  uint32_t *sort_hist, *sort_status;
  size_t status_bytes;
  DevScalars* ds;
  DevScalars h_ds;
  // state machine / errors
  int stage = S_INIT;
  bool poisoned = false;
  char err[512] = "";
  // timing / accounting
  cudaEvent_t ev[SPH_NPHASES][2];
  bool pending[SPH_NPHASES];
  double last_ms[SPH_NPHASES];
  PhaseRow rows[SPH_NPHASES];
  // PHASE accounting (in situ, no phase-edge syncs): a host thread samples the
  // device-written phase tag and the NVML instant power and integrates
  // E_p = sum P dt over the intervals the device spent in phase p.
  struct Acct {
    std::thread th;
    std::atomic<bool> run{false};
    bool active = false;
    std::mutex mu;
    double J[SPH_NPHASES + 1] = {};         // [SPH_NPHASES] = between phases
    double mhz_sum[SPH_NPHASES + 1] = {};
    int64_t mhz_n[SPH_NPHASES + 1] = {};
    int64_t samples = 0;
    double seconds = 0;                     // sampled wall time since reset
    unsigned long long e_start = 0;         // energy counter at reset
    std::chrono::steady_clock::time_point t_start{};
    bool e_start_ok = false;
  } acct;
  Nvml nvml;
  int clock_mode = SPH_CLOCK_DEFAULT;
  unsigned clock_mhz[SPH_NPHASES];
  unsigned current_lock = 0;
  bool locked_any = false;
  bool rec_m_dirty = false;
  uint32_t* last_perm = nullptr;  // the last sort's permutation (SPH_F_ORDER)
  uint8_t* bnd = nullptr;         // per target: a ghost among its neighbours (search)
  uint32_t* perm_saved = nullptr; // its copy while sph_repeat_phase(SORT) reuses the buffers;
                                  // also the inverse permutation of sph_decomp_map
  bool inv_valid = false;         // perm_saved holds the inverse of last_perm
  // SORT: radix passes over digits sort_skip..7 + the run fixup (k_sort.cu);
  // all 8 passes (skip 0) after a step whose fixup met a long run
  int sort_skip = kSortSkipDefault;
  int sort_full_steps = 0;
  int64_t* compact_scratch = nullptr;  // per-block counts of sph_compact / sph_decomp_pack (+ totals)
  int64_t compact_scratch_len = 0;
  Stir stir{};          // turbulence driving (k_stir.cu)
  bool stir_on = false;
  // sph_step as a CUDA graph: one captured step per (buffer parity, sort
  // passes, n); a replay re-applies the host-side effects the capture recorded
  struct StepGraph {
    bool valid = false;
    int cur = 0, skip = 0;
    int64_t n = 0;
    Params P{};          // kernel arguments captured by value: any change -> new capture
    Stir stir{};
    bool stir_on = false;
    cudaGraphExec_t exec = nullptr;
    int cur_after = 0;
    uint32_t* last_perm = nullptr;
    uint64_t* key_sorted = nullptr;
    bool gradh_done = false;
    bool ran[SPH_NPHASES] = {};
    long long launches = 0;
  } graphs[4];
  int graph_next = 0;
  bool graphs_off = false;  // env SPH_NO_GRAPH, or a capture failed
  // DVFS trace (sph_trace_start / sph_trace_stop)
  struct Trace {
    std::thread th;
    std::atomic<bool> run{false};
    bool active = false;
    volatile int* word = nullptr;  // pinned, device-mapped: the running phase
    int* word_dev = nullptr;
    std::vector<sph_trace_sample> buf;
    int64_t taken = 0;
  } trace;
};

namespace {

int fail(sph_ctx* c, int code, const char* fmt, ...) {
  char* buf = c ? c->err : g_err;
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(buf, 512, fmt, ap);
  va_end(ap);
  return code;
}

int cuda_check(sph_ctx* c, cudaError_t e, const char* where) {
  if (e == cudaSuccess) e = cudaGetLastError();
  if (e != cudaSuccess) {
    c->poisoned = true;
    return fail(c, SPH_ERR_CUDA, "%s: %s", where, cudaGetErrorString(e));
  }
  return SPH_OK;
}

int check_ready(sph_ctx* c, int min_stage, const char* what) {
  if (!c) return fail(nullptr, SPH_ERR_ARG, "%s: null context", what);
  if (c->poisoned) return fail(c, SPH_ERR_STATE, "%s: context poisoned by an earlier CUDA error", what);
  if (c->stage < min_stage) return fail(c, SPH_ERR_STATE, "%s: called out of order (stage %d < %d)", what, c->stage, min_stage);
  return SPH_OK;
}

// Row stride of the neighbour-search scratch rows: ngmax + 1 (a spare word for
// the branch-free append) rounded up to 8.
int64_t nrows_ld(const sph_config* cfg) { return ((int64_t)cfg->ngmax + 8) / 8 * 8; }

Fields fields(sph_ctx* c) {
  Fields F;
  F.n = c->n;
  F.cap = c->cfg.n_capacity;
  for (int f = 0; f < kNumStateF; ++f) F.f[f] = c->state[c->cur][f];
  F.id = c->ids[c->cur];
  F.key = c->key_sorted;
  F.rho = c->rho; F.p = c->p; F.c = c->c; F.vol = c->vol; F.prho2 = c->prho2;
  F.wq = c->wq; F.wk = c->wk;
  for (int e = 0; e < 6; ++e) F.C[e] = c->C[e];
  F.ax = c->ax; F.ay = c->ay; F.az = c->az; F.du = c->du;
  F.divv = c->divv; F.bal = c->P.av_switch ? c->bal : nullptr; F.rec_iv = c->rec_iv;
  F.phi = c->phi; F.gcell_start = c->gcell_start; F.gmom = c->gmom;
  F.omega = c->omega; F.vsig = c->vsig;
  for (int a = 0; a < 3; ++a) F.curl[a] = c->curl[a];
  F.nc = c->nc; F.nbr = c->nbr; F.ngmax = c->cfg.ngmax; F.bnd = c->bnd;
  F.nrows = c->nrows; F.nrows_ld = nrows_ld(&c->cfg);
  F.cell_start = c->cell_start;
  F.pos4 = c->pos4;
  F.rec_d = c->rec_d;
  F.rec_i = c->rec_i;
  F.rec_m = c->rec_m;
  F.ds = c->ds;
  return F;
}

void collect_phase(sph_ctx* c, int p) {
  if (!c->pending[p]) return;
  float ms = 0.f;
  if (cudaEventElapsedTime(&ms, c->ev[p][0], c->ev[p][1]) == cudaSuccess) {
    c->rows[p].seconds += ms * 1e-3;
    c->last_ms[p] = ms;
  } else {
    cudaGetLastError();
  }
  c->pending[p] = false;
}

void collect_all(sph_ctx* c) {
  for (int p = 0; p < SPH_NPHASES; ++p) collect_phase(c, p);
}

void apply_clock(sph_ctx* c, int p) {
  if (c->clock_mode == SPH_CLOCK_DEFAULT) return;
  unsigned want = c->clock_mhz[p];
  if (want == 0 || want == c->current_lock) return;
  // The lock applies from the moment NVML sets it, not in stream order: wait
  // until the earlier phases have finished so each runs at its own clock (the
  // wait is part of ManDyn's cost, like the paper's clock-switch latency).
  cudaStreamSynchronize(c->st);
  if (c->nvml.lock_sm_clock(want) == 0) {
    c->current_lock = want;
    c->locked_any = true;
  }
}

__global__ void trace_mark_kernel(int* word, int phase) {
  *(volatile int*)word = phase;
  __threadfence_system();
}

// Tags the DVFS trace with the phase the stream reaches next (trace active only).
void trace_mark(sph_ctx* c, int phase) {
  if (!c->trace.active && !c->acct.active) return;
  trace_mark_kernel<<<1, 1, 0, c->st>>>(c->trace.word_dev, phase);
  note_launch();
}

// The pinned, device-mapped word the trace_mark kernels write: the phase the
// stream is executing (shared by the DVFS trace and PHASE accounting).
int ensure_phase_word(sph_ctx* c) {
  if (c->trace.word) return SPH_OK;
  void* h = nullptr;
  int rc = cuda_check(c, cudaHostAlloc(&h, sizeof(int), cudaHostAllocMapped), "cudaHostAlloc");
  if (rc) return rc;
  void* d = nullptr;
  if ((rc = cuda_check(c, cudaHostGetDevicePointer(&d, h, 0), "cudaHostGetDevicePointer"))) return rc;
  c->trace.word = (volatile int*)h;
  c->trace.word_dev = (int*)d;
  *c->trace.word = -1;
  return SPH_OK;
}

void acct_reset(sph_ctx* c) {
  sph_ctx::Acct& A = c->acct;
  std::lock_guard<std::mutex> g(A.mu);
  for (int p = 0; p <= SPH_NPHASES; ++p) A.J[p] = A.mhz_sum[p] = 0.0, A.mhz_n[p] = 0;
  A.samples = 0;
  A.seconds = 0.0;
  A.e_start_ok = c->nvml.energy_mj(&A.e_start);
  A.t_start = std::chrono::steady_clock::now();
}

// PHASE accounting sampler: every ~0.25 ms the phase tag and the instant power;
// the interval since the previous sample is charged to the phase seen then at
// the power read then (left Riemann sum).  NVML's instant power refreshes about
// every 100 ms on a B200 (profiles/r02_probe_nvml_instant.json), so the joules
// of a phase shorter than that are its time at the surrounding average power.
int acct_start(sph_ctx* c) {
  if (c->acct.active) return SPH_OK;
  if (!c->nvml.ok) return fail(c, SPH_ERR_NVML, "NVML unavailable: %s", c->nvml.err);
  unsigned probe = 0;
  if (!c->nvml.power_instant_mw(&probe) && !c->nvml.power_mw(&probe))
    return fail(c, SPH_ERR_NVML, "NVML power unreadable: %s", c->nvml.error_string(c->nvml.last_rc));
  int rc = ensure_phase_word(c);
  if (rc) return rc;
  acct_reset(c);
  c->acct.run.store(true);
  c->acct.active = true;
  sph_ctx::Acct* A = &c->acct;
  Nvml* nv = &c->nvml;
  volatile int* word = c->trace.word;
  c->acct.th = std::thread([A, nv, word]() {
    using clk = std::chrono::steady_clock;
    const bool instant = [&] { unsigned v; return nv->power_instant_mw(&v); }();
    auto power = [&](unsigned* v) { return instant ? nv->power_instant_mw(v) : nv->power_mw(v); };
    auto prev = clk::now();
    int ph_prev = *word;
    unsigned p_prev = 0;
    power(&p_prev);
    int64_t k = 0;
    while (A->run.load(std::memory_order_relaxed)) {
      std::this_thread::sleep_for(std::chrono::microseconds(250));
      const auto now = clk::now();
      const int ph = *word;
      unsigned pw = p_prev;
      power(&pw);
      unsigned mhz = 0;
      const bool got_mhz = (++k & 15) == 0 && nv->sm_clock_mhz(&mhz);
      const double dt = std::chrono::duration<double>(now - prev).count();
      const int b = (ph_prev >= 0 && ph_prev < SPH_NPHASES) ? ph_prev : SPH_NPHASES;
      {
        std::lock_guard<std::mutex> g(A->mu);
        A->J[b] += 1e-3 * p_prev * dt;
        A->seconds += dt;
        ++A->samples;
        if (got_mhz) {
          A->mhz_sum[b] += mhz;
          ++A->mhz_n[b];
        }
      }
      prev = now;
      ph_prev = ph;
      p_prev = pw;
    }
  });
  return SPH_OK;
}

void acct_stop(sph_ctx* c) {
  if (!c->acct.active) return;
  c->acct.run.store(false);
  if (c->acct.th.joinable()) c->acct.th.join();
  c->acct.active = false;
}

cudaError_t record_event(sph_ctx* c, cudaEvent_t ev) {
  cudaStreamCaptureStatus cs = cudaStreamCaptureStatusNone;
  cudaStreamIsCapturing(c->st, &cs);
  return cs == cudaStreamCaptureStatusActive ? cudaEventRecordWithFlags(ev, c->st, cudaEventRecordExternal)
                                             : cudaEventRecord(ev, c->st);
}

int phase_begin(sph_ctx* c, int p) {
  trace_mark(c, p);
  if (c->pending[p]) {
    cudaEventSynchronize(c->ev[p][1]);
    collect_phase(c, p);
  }
  apply_clock(c, p);
  c->rows[p].locked = c->current_lock;
  // (External: inside a captured step graph the record is a graph node that
  // records the event when the graph runs, so the phase times stay valid)
  return cuda_check(c, record_event(c, c->ev[p][0]), "cudaEventRecord");
}

int phase_end(sph_ctx* c, int p) {
  int rc = cuda_check(c, record_event(c, c->ev[p][1]), "phase kernels");
  if (rc) return rc;
  trace_mark(c, -1);
  c->pending[p] = true;
  c->rows[p].calls++;
  return SPH_OK;
}

// Reads the device scalars (synchronises) and maps device status bits to codes.
int sync_scalars(sph_ctx* c) {
  int rc = cuda_check(c, cudaMemcpyAsync(&c->h_ds, c->ds, sizeof(DevScalars), cudaMemcpyDeviceToHost, c->st), "scalar copy");
  if (rc) return rc;
  rc = cuda_check(c, cudaStreamSynchronize(c->st), "stream sync");
  if (rc) return rc;
  collect_all(c);
  // sort policy for the next steps: long fixup runs (particles closer than a
  // level-(21 - 8 skip / 3) cell) -> all 8 passes for a while
  if (c->h_ds.sort_maxrun > kSortMaxRun) {
    c->sort_skip = 0;
    c->sort_full_steps = 16;
  } else if (c->sort_full_steps > 0 && --c->sort_full_steps == 0) {
    c->sort_skip = kSortSkipDefault;
  }
  int s = c->h_ds.status;
  if (s & ST_BOX) return fail(c, SPH_ERR_BOX, "degenerate open-axis box (max == min)");
  if (s & ST_CAPACITY)
    return fail(c, SPH_ERR_CAPACITY, "neighbour count %d exceeds ngmax %d", c->h_ds.max_nc, c->cfg.ngmax);
  if (s & ST_SINGULAR) return fail(c, SPH_ERR_SINGULAR, "singular IAD matrix (det <= 0 or non-finite)");
  if (s & ST_DECOMP) return fail(c, SPH_ERR_STATE, "decomposition: a kept/received count differs from the caller's");
  if (s & ST_STIR_NOISE) return fail(c, SPH_ERR_CAPACITY, "driving noise table exhausted (%lld steps)", (long long)c->stir.nsteps);
  return SPH_OK;
}

void fill_stats(sph_ctx* c, sph_nbr_stats* s) {
  if (!s) return;
  s->min_nc = c->n ? c->h_ds.min_nc : 0;
  s->max_nc = c->h_ds.max_nc;
  s->total = (int64_t)c->h_ds.total_nc;
  s->mean_nc = c->n ? (double)c->h_ds.total_nc / (double)c->n : 0.0;
  s->candidates = (int64_t)c->h_ds.cand_total;
  s->passes = (int64_t)c->h_ds.pass_total;
}

__global__ void set_time_kernel(DevScalars* ds, double t, double dt_prev, int first) {
  ds->t = t;
  ds->dt_prev = dt_prev;
  ds->dt = 0.0;
  ds->first = first;
}

__global__ void iota_kernel(int64_t* id, int64_t n) {
  int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (i < n) id[i] = i;
}

__global__ void reset_nbr_stats_kernel(DevScalars* ds) {
  ds->max_nc = 0;
  ds->min_nc = 0x7fffffff;
  ds->total_nc = 0ull;
  ds->cand_total = 0ull;
  ds->pass_total = 0ull;
  ds->status &= ~ST_CAPACITY;
}

// ---- phase bodies (enqueue only) ----
int body_tree(sph_ctx* c) {
  int rc;
  if ((rc = phase_begin(c, SPH_PHASE_KEYS))) return rc;
  launch_reset_scalars(c->ds, c->P, c->st);
  c->key_sorted = c->keyA;
  Fields F = fields(c);
  F.key = c->keyA;
  launch_box_keys(F, c->P, c->st);
  if ((rc = phase_end(c, SPH_PHASE_KEYS))) return rc;

  if ((rc = phase_begin(c, SPH_PHASE_SORT))) return rc;
  uint32_t* perm = nullptr;
  uint64_t* ksorted = nullptr;
  cudaError_t e = launch_sort(F, c->keyA, c->keyB, c->valA, c->valB, c->sort_hist, c->sort_status,
                              c->status_bytes, &perm, &ksorted, c->st, c->sort_skip);
  if ((rc = cuda_check(c, e, "sort"))) return rc;
  c->last_perm = perm;
  c->inv_valid = false;
  const int prv = c->cur;
  c->cur ^= 1;
  c->key_sorted = ksorted;
  launch_permute(fields(c), perm, c->state[prv], c->ids[prv], c->st);
  if ((rc = phase_end(c, SPH_PHASE_SORT))) return rc;

  if ((rc = phase_begin(c, SPH_PHASE_CELLS))) return rc;
  launch_cells(fields(c), c->P, c->level_cap, c->st);
  if ((rc = phase_end(c, SPH_PHASE_CELLS))) return rc;
  c->stage = S_TREE;
  return SPH_OK;
}

int body_neighbors(sph_ctx* c) {
  int rc;
  if ((rc = phase_begin(c, SPH_PHASE_NEIGHBORS))) return rc;
  reset_nbr_stats_kernel<<<1, 1, 0, c->st>>>(c->ds); note_launch();
  launch_neighbors(fields(c), c->P, c->st);
  if ((rc = phase_end(c, SPH_PHASE_NEIGHBORS))) return rc;
  c->stage = S_NBR;
  return SPH_OK;
}

int body_simple(sph_ctx* c, int phase, int next_stage) {
  int rc;
  if ((rc = phase_begin(c, phase))) return rc;
  Fields F = fields(c);
  switch (phase) {
    case SPH_PHASE_DENSITY: launch_density(F, c->P, c->st); break;
    case SPH_PHASE_EOS:
      launch_eos(F, c->P, c->st);
      c->gradh_done = false;
      break;
    case SPH_PHASE_GRADH:
      launch_gradh(F, c->P, c->st);
      if (c->P.ve) launch_eos(F, c->P, c->st, c->P.gradh != 0);  // EOS of the normalised density
      c->gradh_done = true;
      break;
    case SPH_PHASE_IAD: launch_iad(F, c->P, c->st); break;
    case SPH_PHASE_MOMENTUM_ENERGY:
      if (c->rec_m_dirty) {  // ghosts' C were overwritten (sph_set_field)
        launch_refresh_rec_m(F, c->st);
        c->rec_m_dirty = false;
      }
      // (the BOUNDARY half of a split step adds to the INTERIOR half's minimum)
      if (c->P.part != SPH_PART_BOUNDARY)
        cudaMemsetAsync(&c->ds->minhc_ord, 0xff, sizeof(unsigned long long), c->st);
      launch_momentum_energy(F, c->P, c->st);
      break;
    case SPH_PHASE_TIMESTEP: launch_timestep(F, c->P, c->st); break;
    case SPH_PHASE_UPDATE:
      launch_update(F, c->P, c->st);
      launch_advance_time(F, c->st);
      break;
    case SPH_PHASE_STIR: launch_stir(F, c->P, c->stir, c->st); break;
    case SPH_PHASE_GRAVITY: {
      GravParams G{c->cfg.grav_G, c->cfg.grav_eps, c->cfg.grav_theta, c->cfg.grav_level,
                   (c->cfg.grav_theta > 0.0 && !c->cfg.grav_fp64) ? 1 : 0};
      launch_gravity(F, G, c->st);
      break;
    }
  }
  if ((rc = phase_end(c, phase))) return rc;
  c->stage = next_stage;
  return SPH_OK;
}

}  // namespace

// =========================================================================== ABI

extern "C" {

int sph_config_default(sph_config* cfg) {
  if (!cfg) return fail(nullptr, SPH_ERR_ARG, "null config");
  memset(cfg, 0, sizeof(*cfg));
  cfg->n_capacity = 1 << 20;
  for (int a = 0; a < 3; ++a) {
    cfg->box_min[a] = -0.5;
    cfg->box_max[a] = 0.5;
    cfg->periodic[a] = 1;
  }
  cfg->eos = SPH_EOS_IDEAL;
  cfg->gamma = 5.0 / 3.0;
  cfg->cs0 = 1.0;
  cfg->K = 0.79044958943230290;
  cfg->ng0 = 100.0;
  cfg->ngmax = 150;
  cfg->max_cell_level = 8;
  cfg->h_cap = 0.25;
  cfg->k_cour = 0.2;
  cfg->dt_max_growth = 1.1;
  cfg->dt_first = 1e-6;
  cfg->av_alpha = 1.0;
  cfg->av_beta = 2.0;
  cfg->av_eps = 0.01;
  cfg->device = 0;
  cfg->accounting = SPH_ACCOUNTING_OFF;
  cfg->rank = 0;
  cfg->nranks = 1;
  cfg->grav_level = 6;
  cfg->grav_G = 1.0;
  cfg->grav_eps = 0.01;
  cfg->grav_theta = 0.5;
  return SPH_OK;
}

static int validate(const sph_config* c) {
  if (!c) return fail(nullptr, SPH_ERR_ARG, "null config");
  if (c->n_capacity < 1 || c->n_capacity >= (int64_t(1) << 30))
    return fail(nullptr, SPH_ERR_ARG, "n_capacity must be in [1, 2^30)");
  if (c->ngmax < 1 || c->ngmax > 4096) return fail(nullptr, SPH_ERR_ARG, "ngmax must be in [1, 4096]");
  if (c->max_cell_level < 1 || c->max_cell_level > 10) return fail(nullptr, SPH_ERR_ARG, "max_cell_level must be in [1, 10]");
  for (int a = 0; a < 3; ++a)
    if (c->periodic[a] && !(c->box_max[a] > c->box_min[a])) return fail(nullptr, SPH_ERR_ARG, "periodic axis %d: box_max <= box_min", a);
  if (c->eos != SPH_EOS_IDEAL && c->eos != SPH_EOS_ISOTHERMAL) return fail(nullptr, SPH_ERR_ARG, "unknown eos %d", c->eos);
  if (!(c->K > 0) || !(c->dt_first > 0) || !(c->h_cap > 0)) return fail(nullptr, SPH_ERR_ARG, "K, dt_first and h_cap must be > 0");
  if (c->nranks != 1) return fail(nullptr, SPH_ERR_NOT_SUPPORTED, "nranks > 1 is not built into this library version");
  if (c->stir_steps < 0) return fail(nullptr, SPH_ERR_ARG, "stir_steps < 0");
  if (c->divcurl < 0 || c->divcurl > 1 || c->av_switch < 0 || c->av_switch > 1)
    return fail(nullptr, SPH_ERR_ARG, "divcurl and av_switch must be 0 or 1");
  if (c->gradh < 0 || c->gradh > 1 || c->dt_vsig < 0 || c->dt_vsig > 1 || c->ve < 0 || c->ve > 1)
    return fail(nullptr, SPH_ERR_ARG, "gradh, dt_vsig and ve must be 0 or 1");
  if (c->gravity) {
    if (c->periodic[0] || c->periodic[1] || c->periodic[2])
      return fail(nullptr, SPH_ERR_NOT_SUPPORTED, "gravity is for isolated (fully open) boxes");
    if (c->grav_level < 1 || c->grav_level > 8) return fail(nullptr, SPH_ERR_ARG, "grav_level must be in [1, 8]");
    if (!(c->grav_eps >= 0) || !(c->grav_theta >= 0) || !(c->grav_G >= 0))
      return fail(nullptr, SPH_ERR_ARG, "grav_G, grav_eps, grav_theta must be >= 0");
  }
  return SPH_OK;
}

// Computes the arena layout; with ctx != NULL also assigns the slices.
static size_t layout(const sph_config* cfg, char* base, sph_ctx* c) {
  const size_t cap = (size_t)cfg->n_capacity;
  size_t o = 0;
  auto take = [&](size_t bytes) -> char* {
    char* r = base ? base + o : nullptr;
    o += align_up(bytes);
    return r;
  };
  const size_t D = sizeof(double) * cap;
  for (int b = 0; b < 2; ++b) {
    for (int f = 0; f < kNumStateF; ++f) {
      char* p = take(D);
      if (c) c->state[b][f] = (double*)p;
    }
    char* p = take(sizeof(int64_t) * cap);
    if (c) c->ids[b] = (int64_t*)p;
  }
  char* kA = take(sizeof(uint64_t) * cap);
  char* kB = take(sizeof(uint64_t) * cap);
  char* vA = take(sizeof(uint32_t) * cap);
  char* vB = take(sizeof(uint32_t) * cap);
  char* vS = take(sizeof(uint32_t) * cap);  // sph_repeat_phase(SORT) keeps last_perm here
  double** dst[] = {c ? &c->rho : nullptr, c ? &c->p : nullptr, c ? &c->c : nullptr,
                    c ? &c->vol : nullptr, c ? &c->prho2 : nullptr, c ? &c->wq : nullptr,
                    c ? &c->wk : nullptr, c ? &c->ax : nullptr, c ? &c->ay : nullptr,
                    c ? &c->az : nullptr, c ? &c->du : nullptr, c ? &c->divv : nullptr,
                    c ? &c->curl[0] : nullptr, c ? &c->curl[1] : nullptr,
                    c ? &c->curl[2] : nullptr, c ? &c->bal : nullptr};
  for (double** d : dst) {
    char* p = take(D);
    if (c) *d = (double*)p;
  }
  for (int e = 0; e < 6; ++e) {
    char* p = take(D);
    if (c) c->C[e] = (double*)p;
  }
  char* p4 = take(sizeof(float4) * cap);
  char* rd = take(sizeof(Rec4) * cap);
  char* ri = take(sizeof(Rec4) * cap);
  char* rm = take(sizeof(Rec4) * kRecM * cap);
  char* riv = (cfg->divcurl || cfg->av_switch) ? take(sizeof(Rec4) * cap) : nullptr;
  if (c) c->rec_iv = (Rec4*)riv;
  char* om = cfg->gradh ? take(D) : nullptr;
  char* vsg = cfg->dt_vsig ? take(D) : nullptr;
  if (c) {
    c->omega = (double*)om;
    c->vsig = (double*)vsg;
  }
  if (cfg->gravity) {
    const int Lt = cfg->grav_level;
    const size_t ncells = (size_t)((((int64_t)1 << (3 * (Lt + 1))) - 1) / 7);
    char* ph = take(D);
    char* gcs = take(sizeof(uint32_t) * (((size_t)1 << (3 * Lt)) + 1));
    char* gm = take(sizeof(Rec4) * 3 * ncells);
    if (c) {
      c->phi = (double*)ph;
      c->gcell_start = (uint32_t*)gcs;
      c->gmom = (Rec4*)gm;
    }
  }
  if (c) {
    c->pos4 = (float4*)p4;
    c->rec_d = (Rec4*)rd;
    c->rec_i = (Rec4*)ri;
    c->rec_m = (Rec4*)rm;
  }
  char* ncp = take(sizeof(int32_t) * cap);
  char* bndp = take(sizeof(uint8_t) * cap);
  if (c) c->bnd = (uint8_t*)bndp;
  char* nbp = take(sizeof(int32_t) * cap * (size_t)cfg->ngmax);
  char* nrp = take(sizeof(int32_t) * (size_t)kNbrSlots * kNbrSlotRows * (size_t)nrows_ld(cfg));
  const int Lc = level_cap_for(cfg);
  char* cs = take(sizeof(uint32_t) * ((size_t(1) << (3 * Lc)) + 1));
  size_t hb, sb;
  sort_workspace(cfg->n_capacity, &hb, &sb);
  char* hp = take(hb);
  char* sp = take(sb);
  char* dsp = take(sizeof(DevScalars));
  // compaction (blocks + total) and the grouped pack (64 ranks x blocks + total)
  const size_t csl = (size_t)kMaxGhostRanks * ((cap + 1023) / 1024) + 2;
  char* csc = take(sizeof(int64_t) * csl);
  if (c) {
    c->compact_scratch = (int64_t*)csc;
    c->compact_scratch_len = (int64_t)csl;
  }
  const size_t sst = (size_t)cfg->stir_steps;
  char* sA = sst ? take(sizeof(double) * kStirModes * 6) : nullptr;
  char* sB = sst ? take(sizeof(double) * kStirModes * 6) : nullptr;
  char* sw = sst ? take(sizeof(double) * kStirModes) : nullptr;
  char* sn = sst ? take(sizeof(double) * kStirModes * 6 * sst) : nullptr;
  if (c) {
    c->stir.A = (double*)sA;
    c->stir.B = (double*)sB;
    c->stir.w = (double*)sw;
    c->stir.noise = (double*)sn;
  }
  if (c) {
    c->keyA = (uint64_t*)kA; c->keyB = (uint64_t*)kB;
    c->valA = (uint32_t*)vA; c->valB = (uint32_t*)vB; c->perm_saved = (uint32_t*)vS;
    c->nc = (int32_t*)ncp; c->nbr = (int32_t*)nbp; c->nrows = (int32_t*)nrp;
    c->cell_start = (uint32_t*)cs;
    c->level_cap = Lc;
    c->sort_hist = (uint32_t*)hp; c->sort_status = (uint32_t*)sp; c->status_bytes = sb;
    c->ds = (DevScalars*)dsp;
    c->key_sorted = c->keyA;
  }
  return o;
}

int sph_workspace_size(const sph_config* cfg, size_t* bytes) {
  int rc = validate(cfg);
  if (rc) return rc;
  if (!bytes) return fail(nullptr, SPH_ERR_ARG, "null bytes");
  *bytes = layout(cfg, nullptr, nullptr);
  return SPH_OK;
}

int sph_init(const sph_config* cfg, void* arena, size_t arena_bytes, void* stream, sph_ctx** out) {
  int rc = validate(cfg);
  if (rc) return rc;
  if (!out) return fail(nullptr, SPH_ERR_ARG, "null out");
  *out = nullptr;
  size_t need = layout(cfg, nullptr, nullptr);
  if (!arena || arena_bytes < need)
    return fail(nullptr, SPH_ERR_ARG, "arena too small: %zu < %zu bytes", arena_bytes, need);
  if (((uintptr_t)arena) % kAlign) return fail(nullptr, SPH_ERR_ARG, "arena not 256-byte aligned");
  cudaError_t e = cudaSetDevice(cfg->device);
  if (e != cudaSuccess) {
    cudaGetLastError();
    return fail(nullptr, SPH_ERR_CUDA, "cudaSetDevice(%d): %s", cfg->device, cudaGetErrorString(e));
  }
  sph_ctx* c = new (std::nothrow) sph_ctx();
  if (!c) return fail(nullptr, SPH_ERR_ARG, "out of host memory");
  c->cfg = *cfg;
  c->st = (cudaStream_t)stream;
  for (int a = 0; a < 3; ++a) {
    c->P.box_min[a] = cfg->box_min[a];
    c->P.box_max[a] = cfg->box_max[a];
    c->P.periodic[a] = cfg->periodic[a];
  }
  c->P.eos = cfg->eos; c->P.gamma = cfg->gamma; c->P.cs0 = cfg->cs0; c->P.K = cfg->K;
  c->P.ng0 = cfg->ng0; c->P.h_cap = cfg->h_cap; c->P.k_cour = cfg->k_cour;
  c->P.dt_max_growth = cfg->dt_max_growth; c->P.av_alpha = cfg->av_alpha;
  c->P.av_beta = cfg->av_beta; c->P.av_eps = cfg->av_eps; c->P.max_cell_level = cfg->max_cell_level;
  c->P.av_switch = cfg->av_switch ? 1 : 0;
  c->P.divcurl = (cfg->divcurl || cfg->av_switch) ? 1 : 0;
  c->P.gradh = cfg->gradh ? 1 : 0;
  c->P.ve = cfg->ve ? 1 : 0;
  c->P.dt_vsig = cfg->dt_vsig ? 1 : 0;
  c->P.key_box_set = 0;
  c->P.part = SPH_PART_ALL;
  {
    const char* mr = getenv("SPH_NBR_MERGE_RUNS");  // test hook: exercises the merged-run search path
    c->P.nbr_merge_runs = mr ? atoi(mr) : -1;
    const char* ng = getenv("SPH_NO_GRAPH");  // sph_step without its CUDA graph
    c->graphs_off = ng && atoi(ng) != 0;
  }
  layout(cfg, (char*)arena, c);
  for (int p = 0; p < SPH_NPHASES; ++p) {
    c->pending[p] = false;
    c->last_ms[p] = 0;
    c->clock_mhz[p] = 0;
    for (int k = 0; k < 2; ++k) {
      e = cudaEventCreate(&c->ev[p][k]);
      if (e != cudaSuccess) {
        cudaGetLastError();
        delete c;
        return fail(nullptr, SPH_ERR_CUDA, "cudaEventCreate: %s", cudaGetErrorString(e));
      }
    }
  }
  // the arena is the caller's uninitialised memory: every device scalar starts
  // at zero (accumulators such as the decomposition's red_ord are reset only by
  // the kernel that consumes them)
  e = cudaMemsetAsync(c->ds, 0, sizeof(DevScalars), c->st);
  if (e != cudaSuccess) {
    cudaGetLastError();
    delete c;
    return fail(nullptr, SPH_ERR_CUDA, "scalar init: %s", cudaGetErrorString(e));
  }
  launch_reset_scalars(c->ds, c->P, c->st);
  set_time_kernel<<<1, 1, 0, c->st>>>(c->ds, 0.0, cfg->dt_first, 1); note_launch();
  e = cudaStreamSynchronize(c->st);
  if (e == cudaSuccess) e = cudaGetLastError();
  if (e != cudaSuccess) {
    fail(nullptr, SPH_ERR_CUDA, "init kernels: %s", cudaGetErrorString(e));
    delete c;
    return SPH_ERR_CUDA;
  }
  c->nvml.init(cfg->device);  // failure only disables energy/clock features
  c->stage = S_INIT;
  // PHASE accounting from the start: without NVML the energy rows stay
  // unavailable (NVML errors never fail or poison)
  if (cfg->accounting == SPH_ACCOUNTING_PHASE && acct_start(c) != SPH_OK) c->err[0] = 0;
  *out = c;
  return SPH_OK;
}

void sph_finalize(sph_ctx* c) {
  if (!c) return;
  if (c->trace.active) sph_trace_stop(c, nullptr, 0, nullptr);
  acct_stop(c);
  if (c->trace.word) cudaFreeHost((void*)c->trace.word);
  if (c->locked_any) c->nvml.reset_sm_clock();
  c->nvml.shutdown();
  if (!c->poisoned) cudaStreamSynchronize(c->st);
  for (int p = 0; p < SPH_NPHASES; ++p)
    for (int k = 0; k < 2; ++k) cudaEventDestroy(c->ev[p][k]);
  for (auto& g : c->graphs)
    if (g.exec) cudaGraphExecDestroy(g.exec);
  cudaGetLastError();
  delete c;
}

const char* sph_last_error(const sph_ctx* c) { return c ? c->err : g_err; }

const char* sph_phase_name(int p) {
  return (p >= 0 && p < SPH_NPHASES) ? kPhaseNames[p] : "unknown";
}

int sph_set_particles(sph_ctx* c, int64_t n, const double* x, const double* y, const double* z,
                      const double* vx, const double* vy, const double* vz, const double* h,
                      const double* m, const double* u, const double* du_m1, const int64_t* id,
                      int mem) {
  int rc = check_ready(c, S_INIT, "sph_set_particles");
  if (rc) return rc;
  if (n < 0) return fail(c, SPH_ERR_ARG, "n < 0");
  if (n > c->cfg.n_capacity) return fail(c, SPH_ERR_CAPACITY, "n = %lld exceeds n_capacity %lld", (long long)n, (long long)c->cfg.n_capacity);
  if (mem != SPH_MEM_HOST && mem != SPH_MEM_DEVICE) return fail(c, SPH_ERR_ARG, "mem must be HOST or DEVICE");
  const double* src[kNumStateF] = {x, y, z, vx, vy, vz, h, m, u, du_m1};
  for (int f = 0; f < kNumStateF - 1; ++f)
    if (n > 0 && !src[f]) return fail(c, SPH_ERR_ARG, "null particle array %d", f);
  const cudaMemcpyKind kind = mem == SPH_MEM_HOST ? cudaMemcpyHostToDevice : cudaMemcpyDeviceToDevice;
  c->n = n;
  if (n > 0) {
    for (int f = 0; f < kNumStateF; ++f) {
      if (src[f]) rc = cuda_check(c, cudaMemcpyAsync(c->state[c->cur][f], src[f], sizeof(double) * n, kind, c->st), "particle copy");
      else rc = cuda_check(c, cudaMemsetAsync(c->state[c->cur][f], 0, sizeof(double) * n, c->st), "memset");
      if (rc) return rc;
    }
    if (id) rc = cuda_check(c, cudaMemcpyAsync(c->ids[c->cur], id, sizeof(int64_t) * n, kind, c->st), "id copy");
    else {
      iota_kernel<<<(unsigned)div_up(n, 256), 256, 0, c->st>>>(c->ids[c->cur], n); note_launch();
      rc = cuda_check(c, cudaSuccess, "iota");
    }
    if (rc) return rc;
  }
  c->stage = S_PART;
  return SPH_OK;
}

int sph_set_time(sph_ctx* c, double t, double dt_prev, int first_step) {
  int rc = check_ready(c, S_INIT, "sph_set_time");
  if (rc) return rc;
  if (!(dt_prev > 0)) return fail(c, SPH_ERR_ARG, "dt_prev must be > 0");
  set_time_kernel<<<1, 1, 0, c->st>>>(c->ds, t, dt_prev, first_step ? 1 : 0); note_launch();
  return cuda_check(c, cudaSuccess, "set_time");
}

int sph_get_time(sph_ctx* c, double* t, double* dt_prev, int* first_step) {
  int rc = check_ready(c, S_INIT, "sph_get_time");
  if (rc) return rc;
  rc = cuda_check(c, cudaMemcpyAsync(&c->h_ds, c->ds, sizeof(DevScalars), cudaMemcpyDeviceToHost, c->st), "copy");
  if (!rc) rc = cuda_check(c, cudaStreamSynchronize(c->st), "sync");
  if (rc) return rc;
  if (t) *t = c->h_ds.t;
  if (dt_prev) *dt_prev = c->h_ds.dt_prev;
  if (first_step) *first_step = c->h_ds.first;
  return SPH_OK;
}

int sph_get_n(const sph_ctx* c, int64_t* n) {
  if (!c || !n) return fail(nullptr, SPH_ERR_ARG, "null argument");
  *n = c->n;
  return SPH_OK;
}

int sph_get_field(sph_ctx* c, int field, void* dst, int mem) {
  int rc = check_ready(c, S_INIT, "sph_get_field");
  if (rc) return rc;
  if (!dst && c->n > 0) return fail(c, SPH_ERR_ARG, "null dst");
  if (mem != SPH_MEM_HOST && mem != SPH_MEM_DEVICE && mem != SPH_MEM_HOST_ASYNC)
    return fail(c, SPH_ERR_ARG, "mem must be HOST, DEVICE or HOST_ASYNC");
  const void* src = nullptr;
  size_t esz = sizeof(double);
  if (field >= SPH_F_X && field <= SPH_F_DU_M1) src = c->state[c->cur][field - SPH_F_X];
  else if (field == SPH_F_ID) { src = c->ids[c->cur]; esz = 8; }
  else if (field == SPH_F_KEY) { src = c->key_sorted; esz = 8; }
  else if (field == SPH_F_NC) { src = c->nc; esz = 4; }
  else if (field == SPH_F_RHO) src = c->rho;
  else if (field == SPH_F_P) src = c->p;
  else if (field == SPH_F_C) src = c->c;
  else if (field >= SPH_F_C11 && field <= SPH_F_C33) src = c->C[field - SPH_F_C11];
  else if (field == SPH_F_AX) src = c->ax;
  else if (field == SPH_F_AY) src = c->ay;
  else if (field == SPH_F_AZ) src = c->az;
  else if (field == SPH_F_DU) src = c->du;
  else if (field == SPH_F_DIVV) src = c->divv;
  else if (field >= SPH_F_CURLX && field <= SPH_F_CURLZ) src = c->curl[field - SPH_F_CURLX];
  else if (field == SPH_F_BAL) src = c->bal;
  else if (field == SPH_F_PHI) {
    if (!c->phi) return fail(c, SPH_ERR_ARG, "SPH_F_PHI needs cfg.gravity");
    src = c->phi;
  }
  else if (field == SPH_F_OMEGA) {
    if (!c->omega) return fail(c, SPH_ERR_ARG, "SPH_F_OMEGA needs cfg.gradh");
    src = c->omega;
  }
  else if (field == SPH_F_VSIG) {
    if (!c->vsig) return fail(c, SPH_ERR_ARG, "SPH_F_VSIG needs cfg.dt_vsig");
    src = c->vsig;
  }
  else if (field == SPH_F_ORDER) {
    if (!c->last_perm || c->stage < S_TREE) return fail(c, SPH_ERR_STATE, "SPH_F_ORDER needs sph_build_tree");
    src = c->last_perm;
    esz = 4;
  }
  else return fail(c, SPH_ERR_ARG, "unknown field %d", field);
  if (c->n == 0) return SPH_OK;
  const cudaMemcpyKind kind = mem == SPH_MEM_DEVICE ? cudaMemcpyDeviceToDevice : cudaMemcpyDeviceToHost;
  rc = cuda_check(c, cudaMemcpyAsync(dst, src, esz * c->n, kind, c->st), "field copy");
  if (rc || mem == SPH_MEM_HOST_ASYNC) return rc;  // valid after sph_sync (pinned dst: overlaps)
  rc = cuda_check(c, cudaStreamSynchronize(c->st), "sync");
  if (!rc) collect_all(c);
  return rc;
}

int sph_sync(sph_ctx* c) {
  int rc = check_ready(c, S_INIT, "sph_sync");
  if (rc) return rc;
  rc = cuda_check(c, cudaStreamSynchronize(c->st), "sync");
  if (!rc) collect_all(c);
  return rc;
}

int sph_set_field(sph_ctx* c, int field, const void* src, int mem) {
  int rc = check_ready(c, S_INIT, "sph_set_field");
  if (rc) return rc;
  if (!src && c->n > 0) return fail(c, SPH_ERR_ARG, "null src");
  if (mem != SPH_MEM_HOST && mem != SPH_MEM_DEVICE) return fail(c, SPH_ERR_ARG, "mem must be HOST or DEVICE");
  double* dst = nullptr;
  if (field == SPH_F_RHO) {
    if (c->stage < S_DENS) return fail(c, SPH_ERR_STATE, "sph_set_field(RHO) before sph_density");
    dst = c->rho;
  } else if (field >= SPH_F_C11 && field <= SPH_F_C33) {
    if (c->stage < S_IAD) return fail(c, SPH_ERR_STATE, "sph_set_field(C) before sph_iad");
    dst = c->C[field - SPH_F_C11];
    c->rec_m_dirty = true;
  } else if (field == SPH_F_BAL && c->P.av_switch) {
    if (c->stage < S_IAD) return fail(c, SPH_ERR_STATE, "sph_set_field(BAL) before sph_iad");
    dst = c->bal;
    c->rec_m_dirty = true;
  } else if (field == SPH_F_OMEGA && c->omega) {
    // owners' Omega over the ghosts (multi-GPU halo): p/(Omega rho^2) follows
    if (!c->gradh_done || c->stage != S_EOS)
      return fail(c, SPH_ERR_STATE, "sph_set_field(OMEGA) must follow sph_gradh, before sph_iad");
    if (c->n == 0) return SPH_OK;
    const cudaMemcpyKind k2 = mem == SPH_MEM_HOST ? cudaMemcpyHostToDevice : cudaMemcpyDeviceToDevice;
    rc = cuda_check(c, cudaMemcpyAsync(c->omega, src, sizeof(double) * c->n, k2, c->st), "set field");
    if (rc) return rc;
    launch_prho2(fields(c), c->st);
    return cuda_check(c, cudaGetLastError(), "prho2");
  } else {
    return fail(c, SPH_ERR_ARG, "field %d is not settable", field);
  }
  if (c->n == 0) return SPH_OK;
  const cudaMemcpyKind kind = mem == SPH_MEM_HOST ? cudaMemcpyHostToDevice : cudaMemcpyDeviceToDevice;
  rc = cuda_check(c, cudaMemcpyAsync(dst, src, sizeof(double) * c->n, kind, c->st), "set field");
  if (rc || !(field == SPH_F_RHO && c->P.ve && c->gradh_done && c->stage == S_EOS)) return rc;
  launch_eos(fields(c), c->P, c->st, c->P.gradh != 0);  // owners' normalised rho (reading 23)
  return cuda_check(c, cudaGetLastError(), "eos refresh");
}

int sph_get_local_min_hc(sph_ctx* c, double* min_hc) {
  int rc = check_ready(c, S_MOM, "sph_get_local_min_hc");
  if (rc) return rc;
  if (!min_hc) return fail(c, SPH_ERR_ARG, "null min_hc");
  rc = cuda_check(c, cudaMemcpyAsync(&c->h_ds, c->ds, sizeof(DevScalars), cudaMemcpyDeviceToHost, c->st), "copy");
  if (!rc) rc = cuda_check(c, cudaStreamSynchronize(c->st), "sync");
  if (rc) return rc;
  const unsigned long long o = c->h_ds.minhc_ord;
  if (o == ~0ull) {
    *min_hc = INFINITY;
  } else {
    const unsigned long long b = (o >> 63) ? (o & 0x7fffffffffffffffull) : ~o;
    memcpy(min_hc, &b, sizeof(double));
  }
  return SPH_OK;
}

__global__ void set_minhc_kernel(DevScalars* ds, unsigned long long o) { ds->minhc_ord = o; }

int sph_set_global_min_hc(sph_ctx* c, double min_hc) {
  int rc = check_ready(c, S_MOM, "sph_set_global_min_hc");
  if (rc) return rc;
  if (!(min_hc > 0)) return fail(c, SPH_ERR_ARG, "min_hc must be > 0");
  unsigned long long b;
  memcpy(&b, &min_hc, sizeof(double));
  const unsigned long long o = b | 0x8000000000000000ull;  // order-preserving code of a positive double
  set_minhc_kernel<<<1, 1, 0, c->st>>>(c->ds, o);
  note_launch();
  return cuda_check(c, cudaSuccess, "set_minhc");
}

// ---------------------------------------------------------------- decomposition plumbing
int sph_compute_keys(sph_ctx* c) {
  int rc = check_ready(c, S_PART, "sph_compute_keys");
  if (rc) return rc;
  if ((rc = phase_begin(c, SPH_PHASE_KEYS))) return rc;
  launch_reset_scalars(c->ds, c->P, c->st);
  Fields F = fields(c);
  F.key = c->keyA;
  launch_box_keys(F, c->P, c->st);
  c->key_sorted = c->keyA;  // keys of the current (unsorted) order
  if ((rc = phase_end(c, SPH_PHASE_KEYS))) return rc;
  c->stage = S_PART;
  return SPH_OK;
}

int sph_compact(sph_ctx* c, const uint8_t* keep, int drop_ghosts, int64_t* n_out) {
  int rc = check_ready(c, S_PART, "sph_compact");
  if (rc) return rc;
  const int nxt = c->cur ^ 1;
  int64_t* total = c->compact_scratch + (c->cfg.n_capacity + 1023) / 1024 + 1;
  rc = cuda_check(c, launch_compact(c->n, keep, drop_ghosts ? 1 : 0, c->state[c->cur], c->ids[c->cur],
                                    c->state[nxt], c->ids[nxt], c->compact_scratch, total, c->st),
                  "compact");
  if (rc) return rc;
  int64_t n = 0;
  rc = cuda_check(c, cudaMemcpyAsync(&n, total, sizeof(int64_t), cudaMemcpyDeviceToHost, c->st), "copy");
  if (!rc) rc = cuda_check(c, cudaStreamSynchronize(c->st), "sync");
  if (rc) return rc;
  c->cur = nxt;
  c->n = n;
  c->stage = S_PART;
  if (n_out) *n_out = n;
  return SPH_OK;
}

int sph_pack_rows(sph_ctx* c, const int64_t* idx, int64_t m, uint64_t or_id, double* dst) {
  int rc = check_ready(c, S_PART, "sph_pack_rows");
  if (rc) return rc;
  if (m < 0 || (m > 0 && (!idx || !dst))) return fail(c, SPH_ERR_ARG, "bad idx/dst");
  return cuda_check(c, launch_pack_rows(m, idx, c->state[c->cur], c->ids[c->cur], or_id, dst, c->st), "pack");
}

int sph_append_rows(sph_ctx* c, const double* rows, int64_t m) {
  int rc = check_ready(c, S_PART, "sph_append_rows");
  if (rc) return rc;
  if (m < 0 || (m > 0 && !rows)) return fail(c, SPH_ERR_ARG, "bad rows");
  if (c->n + m > c->cfg.n_capacity)
    return fail(c, SPH_ERR_CAPACITY, "n + m = %lld exceeds n_capacity %lld", (long long)(c->n + m), (long long)c->cfg.n_capacity);
  rc = cuda_check(c, launch_append_rows(m, c->n, rows, c->state[c->cur], c->ids[c->cur], c->st), "append");
  if (rc) return rc;
  c->n += m;
  c->stage = S_PART;
  return SPH_OK;
}

int sph_select_ghosts(sph_ctx* c, const double* boxes, int R, int self, double radius, uint64_t* mask) {
  int rc = check_ready(c, S_PART, "sph_select_ghosts");
  if (rc) return rc;
  if (R < 1 || R > kMaxGhostRanks || !boxes || (c->n > 0 && !mask)) return fail(c, SPH_ERR_ARG, "bad boxes/R/mask");
  double L[3];
  int per[3];
  for (int a = 0; a < 3; ++a) {
    L[a] = c->cfg.box_max[a] - c->cfg.box_min[a];
    per[a] = c->cfg.periodic[a];
  }
  return cuda_check(c, launch_select_ghosts(c->n, c->state[c->cur], boxes, R, self, radius, L, per, mask, c->st),
                    "select ghosts");
}

static double* double_field(sph_ctx* c, int field) {
  if (field >= SPH_F_X && field <= SPH_F_DU_M1) return c->state[c->cur][field - SPH_F_X];
  switch (field) {
    case SPH_F_RHO: return c->rho;
    case SPH_F_P: return c->p;
    case SPH_F_C: return c->c;
    case SPH_F_C11: case SPH_F_C12: case SPH_F_C13: case SPH_F_C22: case SPH_F_C23: case SPH_F_C33:
      return c->C[field - SPH_F_C11];
    case SPH_F_AX: return c->ax;
    case SPH_F_AY: return c->ay;
    case SPH_F_AZ: return c->az;
    case SPH_F_DU: return c->du;
    case SPH_F_DIVV: return c->divv;
    case SPH_F_CURLX: case SPH_F_CURLY: case SPH_F_CURLZ: return c->curl[field - SPH_F_CURLX];
    case SPH_F_BAL: return c->bal;
    case SPH_F_PHI: return c->phi;
    case SPH_F_OMEGA: return c->omega;
    case SPH_F_VSIG: return c->vsig;
    default: return nullptr;
  }
}

int sph_gather_field(sph_ctx* c, int field, const int64_t* idx, int64_t m, double* dst) {
  int rc = check_ready(c, S_INIT, "sph_gather_field");
  if (rc) return rc;
  double* f = double_field(c, field);
  if (!f) return fail(c, SPH_ERR_ARG, "field %d is not a double field of this configuration", field);
  if (m < 0 || (m > 0 && (!idx || !dst))) return fail(c, SPH_ERR_ARG, "bad idx/dst");
  return cuda_check(c, launch_gather_field(m, idx, f, dst, c->st), "gather");
}

int sph_scatter_field(sph_ctx* c, int field, const int64_t* idx, int64_t m, const double* src) {
  int rc = check_ready(c, S_INIT, "sph_scatter_field");
  if (rc) return rc;
  if (m < 0 || (m > 0 && (!idx || !src))) return fail(c, SPH_ERR_ARG, "bad idx/src");
  double* f = nullptr;
  bool prho2 = false;
  bool eos_refresh = false;
  if (field == SPH_F_RHO) {
    if (c->stage < S_DENS) return fail(c, SPH_ERR_STATE, "scatter(RHO) before sph_density");
    f = c->rho;
    // after a volume-element GRADH the EOS already ran: run it again on the
    // owners' normalised densities (reading 23)
    eos_refresh = c->P.ve && c->gradh_done && c->stage == S_EOS;
  } else if (field >= SPH_F_C11 && field <= SPH_F_C33) {
    if (c->stage < S_IAD) return fail(c, SPH_ERR_STATE, "scatter(C) before sph_iad");
    f = c->C[field - SPH_F_C11];
    c->rec_m_dirty = true;
  } else if (field == SPH_F_BAL && c->P.av_switch) {
    if (c->stage < S_IAD) return fail(c, SPH_ERR_STATE, "scatter(BAL) before sph_iad");
    f = c->bal;
    c->rec_m_dirty = true;
  } else if (field == SPH_F_OMEGA && c->omega) {
    if (!c->gradh_done || c->stage != S_EOS)
      return fail(c, SPH_ERR_STATE, "scatter(OMEGA) must follow sph_gradh, before sph_iad");
    f = c->omega;
    prho2 = true;
  } else {
    return fail(c, SPH_ERR_ARG, "field %d is not settable", field);
  }
  rc = cuda_check(c, launch_scatter_field(m, idx, src, f, c->st), "scatter");
  if (rc) return rc;
  if (eos_refresh) {
    launch_eos(fields(c), c->P, c->st, c->P.gradh != 0);
    return cuda_check(c, cudaGetLastError(), "eos refresh");
  }
  if (!prho2) return rc;
  launch_prho2(fields(c), c->st);
  return cuda_check(c, cudaGetLastError(), "prho2");
}

// ---------------------------------------------------------------- SFC decomposition (device)
int sph_decomp_reduce(sph_ctx* c, double* red) {
  int rc = check_ready(c, S_PART, "sph_decomp_reduce");
  if (rc) return rc;
  if (!red) return fail(c, SPH_ERR_ARG, "null red");
  return cuda_check(c, launch_decomp_reduce(c->n, c->state[c->cur], c->ids[c->cur], c->ds->red_ord, red, c->st),
                    "decomp reduce");
}

int sph_set_key_box(sph_ctx* c, const double* red) {
  int rc = check_ready(c, S_INIT, "sph_set_key_box");
  if (rc) return rc;
  if (!red) {
    c->P.key_box_set = 0;
    return SPH_OK;
  }
  rc = cuda_check(c, cudaMemcpyAsync(c->ds->key_box, red, sizeof(double) * 7, cudaMemcpyDeviceToDevice, c->st),
                  "key box");
  if (!rc) c->P.key_box_set = 1;
  return rc;
}

int sph_key_histogram(sph_ctx* c, int bits, int64_t* hist) {
  int rc = check_ready(c, S_PART, "sph_key_histogram");
  if (rc) return rc;
  if (bits < 3 || bits > 21 || bits % 3 || !hist) return fail(c, SPH_ERR_ARG, "bits must be a multiple of 3 in [3, 21]");
  if (c->key_sorted != c->keyA) return fail(c, SPH_ERR_STATE, "sph_key_histogram needs sph_compute_keys");
  return cuda_check(c, launch_key_histogram(c->n, c->keyA, c->ids[c->cur], bits, hist, c->st), "key histogram");
}

int sph_decomp_owners(sph_ctx* c, const int64_t* hist, int bits, int rank, int world, uint64_t* mig_mask,
                      int64_t* counts) {
  int rc = check_ready(c, S_PART, "sph_decomp_owners");
  if (rc) return rc;
  if (bits < 3 || bits > 21 || bits % 3 || !hist || !counts || (c->n > 0 && !mig_mask))
    return fail(c, SPH_ERR_ARG, "bad bits / buffers");
  if (world < 1 || world > kMaxGhostRanks || rank < 0 || rank >= world) return fail(c, SPH_ERR_ARG, "bad rank/world");
  if (c->key_sorted != c->keyA) return fail(c, SPH_ERR_STATE, "sph_decomp_owners needs sph_compute_keys");
  return cuda_check(c, launch_decomp_owners(c->n, c->keyA, c->ids[c->cur], hist, bits, rank, world, c->ds->splits,
                                            mig_mask, counts, c->st), "decomp owners");
}

int sph_decomp_ghosts(sph_ctx* c, int bits, int rank, int world, uint64_t* mask, int64_t* counts) {
  int rc = check_ready(c, S_PART, "sph_decomp_ghosts");
  if (rc) return rc;
  if (bits < 3 || bits > 21 || bits % 3 || !counts || (c->n > 0 && !mask)) return fail(c, SPH_ERR_ARG, "bad bits / buffers");
  if (world < 1 || world > kMaxGhostRanks || rank < 0 || rank >= world) return fail(c, SPH_ERR_ARG, "bad rank/world");
  if (!c->P.key_box_set) return fail(c, SPH_ERR_STATE, "sph_decomp_ghosts needs sph_set_key_box (global h_max)");
  if (c->key_sorted != c->keyA) return fail(c, SPH_ERR_STATE, "sph_decomp_ghosts needs sph_compute_keys");
  return cuda_check(c, launch_decomp_ghosts(c->n, c->keyA, bits, rank, world, c->ds->splits, c->ds, c->P, mask,
                                            counts, c->st), "decomp ghosts");
}

int sph_decomp_pack(sph_ctx* c, const uint64_t* mask, int world, uint64_t or_id, double* rows, int64_t* pos) {
  int rc = check_ready(c, S_PART, "sph_decomp_pack");
  if (rc) return rc;
  if (world < 1 || world > kMaxGhostRanks || (c->n > 0 && (!mask || !rows || !pos))) return fail(c, SPH_ERR_ARG, "bad buffers");
  int64_t* total = c->compact_scratch + c->compact_scratch_len - 1;
  const int64_t nb = div_up(c->n, 1024);
  if (nb * world + 1 > c->compact_scratch_len) return fail(c, SPH_ERR_CAPACITY, "pack scratch too small");
  return cuda_check(c, launch_route_pack(c->n, mask, world, c->state[c->cur], c->ids[c->cur], or_id, rows, pos,
                                         c->compact_scratch, total, c->st), "decomp pack");
}

__global__ void check_count_kernel(const int64_t* total, int64_t expected, DevScalars* ds) {
  if (*total != expected) ds->status |= ST_DECOMP;
}

int sph_decomp_drop(sph_ctx* c, const uint64_t* drop_mask, int64_t n_expected) {
  int rc = check_ready(c, S_PART, "sph_decomp_drop");
  if (rc) return rc;
  if (n_expected < 0 || n_expected > c->n) return fail(c, SPH_ERR_ARG, "n_expected out of range");
  c->stage = S_PART;
  if (n_expected == c->n) return SPH_OK;  // the caller's counts say nothing goes
  const int nxt = c->cur ^ 1;
  int64_t* total = c->compact_scratch + (c->cfg.n_capacity + 1023) / 1024 + 1;
  // the ghosts (SPH_GHOST_BIT) and the particles with drop_mask[i] != 0 go
  rc = cuda_check(c, launch_compact(c->n, nullptr, 1, c->state[c->cur], c->ids[c->cur], c->state[nxt],
                                    c->ids[nxt], c->compact_scratch, total, c->st, drop_mask), "decomp drop");
  if (rc) return rc;
  check_count_kernel<<<1, 1, 0, c->st>>>(total, n_expected, c->ds);
  note_launch();
  c->cur = nxt;
  c->n = n_expected;  // the caller's count (known from the routed counts): no sync
  return cuda_check(c, cudaGetLastError(), "check count");
}

int sph_decomp_map(sph_ctx* c, const int64_t* pre, int64_t first, int64_t m, int64_t* post) {
  int rc = check_ready(c, S_TREE, "sph_decomp_map");
  if (rc) return rc;
  if (m < 0 || (m > 0 && !post) || (!pre && (first < 0 || first + m > c->n))) return fail(c, SPH_ERR_ARG, "bad map arguments");
  if (!c->inv_valid) {
    if ((rc = cuda_check(c, launch_inverse_perm(c->n, c->last_perm, c->perm_saved, c->st), "inverse perm"))) return rc;
    c->inv_valid = true;
  }
  return cuda_check(c, launch_map_positions(m, pre, first, c->perm_saved, post, c->st), "map positions");
}

static int halo_fields(sph_ctx* c, const int32_t* flds, int nf, double** f, bool for_scatter, bool* dirty_rec,
                       bool* prho2, bool* eos) {
  if (nf < 1 || nf > 16 || !flds) return fail(c, SPH_ERR_ARG, "1..16 fields");
  for (int q = 0; q < nf; ++q) {
    const int fd = flds[q];
    f[q] = double_field(c, fd);
    if (!f[q]) return fail(c, SPH_ERR_ARG, "field %d is not a double field of this configuration", fd);
    if (!for_scatter) continue;
    if (fd == SPH_F_RHO) {
      if (c->stage < S_DENS) return fail(c, SPH_ERR_STATE, "halo(RHO) before sph_density");
      *eos = *eos || (c->P.ve && c->gradh_done && c->stage == S_EOS);
    } else if ((fd >= SPH_F_C11 && fd <= SPH_F_C33) || (fd == SPH_F_BAL && c->P.av_switch)) {
      if (c->stage < S_IAD) return fail(c, SPH_ERR_STATE, "halo(C/BAL) before sph_iad");
      *dirty_rec = true;
    } else if (fd == SPH_F_OMEGA && c->omega) {
      if (!c->gradh_done || c->stage != S_EOS) return fail(c, SPH_ERR_STATE, "halo(OMEGA) must follow sph_gradh, before sph_iad");
      *prho2 = true;
    } else {
      return fail(c, SPH_ERR_ARG, "field %d is not settable", fd);
    }
  }
  return SPH_OK;
}

int sph_halo_gather(sph_ctx* c, const int32_t* flds, int nf, const int64_t* idx, int64_t m, double* dst) {
  int rc = check_ready(c, S_INIT, "sph_halo_gather");
  if (rc) return rc;
  if (m < 0 || (m > 0 && (!idx || !dst))) return fail(c, SPH_ERR_ARG, "bad idx/dst");
  double* f[16];
  bool a = false, b = false, e = false;
  if ((rc = halo_fields(c, flds, nf, f, false, &a, &b, &e))) return rc;
  return cuda_check(c, launch_halo(m, idx, f, nf, dst, true, c->st), "halo gather");
}

int sph_halo_scatter(sph_ctx* c, const int32_t* flds, int nf, const int64_t* idx, int64_t m, const double* src) {
  int rc = check_ready(c, S_INIT, "sph_halo_scatter");
  if (rc) return rc;
  if (m < 0 || (m > 0 && (!idx || !src))) return fail(c, SPH_ERR_ARG, "bad idx/src");
  double* f[16];
  bool dirty = false, prho2 = false, eos = false;
  if ((rc = halo_fields(c, flds, nf, f, true, &dirty, &prho2, &eos))) return rc;
  if ((rc = cuda_check(c, launch_halo(m, idx, f, nf, const_cast<double*>(src), false, c->st), "halo scatter"))) return rc;
  if (dirty) c->rec_m_dirty = true;
  if (eos) launch_eos(fields(c), c->P, c->st, c->P.gradh != 0);  // owners' normalised rho (reading 23)
  if (prho2) launch_prho2(fields(c), c->st);
  return cuda_check(c, cudaGetLastError(), "halo refresh");
}

__global__ void min_hc_get_kernel(const DevScalars* ds, double* out) {
  const unsigned long long o = ds->minhc_ord;
  *out = o == ~0ull ? INFINITY : unord(o);
}
__global__ void min_hc_set_kernel(DevScalars* ds, const double* in) { ds->minhc_ord = ord_of(*in); }

int sph_min_hc_dev(sph_ctx* c, double* dst) {
  int rc = check_ready(c, S_MOM, "sph_min_hc_dev");
  if (rc) return rc;
  if (!dst) return fail(c, SPH_ERR_ARG, "null dst");
  min_hc_get_kernel<<<1, 1, 0, c->st>>>(c->ds, dst);
  note_launch();
  return cuda_check(c, cudaGetLastError(), "min hc");
}

int sph_set_min_hc_dev(sph_ctx* c, const double* src) {
  int rc = check_ready(c, S_MOM, "sph_set_min_hc_dev");
  if (rc) return rc;
  if (!src) return fail(c, SPH_ERR_ARG, "null src");
  min_hc_set_kernel<<<1, 1, 0, c->st>>>(c->ds, src);
  note_launch();
  return cuda_check(c, cudaGetLastError(), "set min hc");
}

int sph_build_tree(sph_ctx* c) {
  int rc = check_ready(c, S_PART, "sph_build_tree");
  if (rc) return rc;
  return body_tree(c);
}

int sph_find_neighbors(sph_ctx* c, sph_nbr_stats* stats) {
  int rc = check_ready(c, S_TREE, "sph_find_neighbors");
  if (rc) return rc;
  if ((rc = body_neighbors(c))) return rc;
  if (!stats) return SPH_OK;
  rc = sync_scalars(c);
  fill_stats(c, stats);
  return rc;
}

int sph_get_neighbors(sph_ctx* c, int64_t* offsets, int32_t* idx, int64_t idx_cap) {
  int rc = check_ready(c, S_NBR, "sph_get_neighbors");
  if (rc) return rc;
  if (!offsets) return fail(c, SPH_ERR_ARG, "null offsets");
  const int64_t n = c->n;
  std::vector<int32_t> nc((size_t)n);
  if (n) {
    rc = cuda_check(c, cudaMemcpyAsync(nc.data(), c->nc, 4 * n, cudaMemcpyDeviceToHost, c->st), "nc copy");
    if (!rc) rc = cuda_check(c, cudaStreamSynchronize(c->st), "sync");
    if (rc) return rc;
  }
  offsets[0] = 0;
  int maxnc = 0;
  for (int64_t i = 0; i < n; ++i) {
    int k = std::min(nc[i], c->cfg.ngmax);
    maxnc = std::max(maxnc, k);
    offsets[i + 1] = offsets[i] + k;
  }
  if (offsets[n] > idx_cap || (!idx && offsets[n] > 0))
    return fail(c, SPH_ERR_CAPACITY, "idx_cap %lld < %lld neighbours", (long long)idx_cap, (long long)offsets[n]);
  if (maxnc == 0) return SPH_OK;
  std::vector<int32_t> rows((size_t)maxnc * n);
  rc = cuda_check(c, cudaMemcpy2DAsync(rows.data(), 4 * n, c->nbr, 4 * c->cfg.n_capacity, 4 * n, maxnc, cudaMemcpyDeviceToHost, c->st), "list copy");
  if (!rc) rc = cuda_check(c, cudaStreamSynchronize(c->st), "sync");
  if (rc) return rc;
  for (int64_t i = 0; i < n; ++i)
    for (int64_t k = 0; k < offsets[i + 1] - offsets[i]; ++k) idx[offsets[i] + k] = rows[(size_t)k * n + i];
  return SPH_OK;
}

int sph_get_neighbor_rows(sph_ctx* c, const int64_t* targets, int64_t nt, int64_t* offsets,
                          int32_t* idx, int64_t idx_cap) {
  int rc = check_ready(c, S_NBR, "sph_get_neighbor_rows");
  if (rc) return rc;
  if (nt < 0 || (nt > 0 && (!targets || !offsets))) return fail(c, SPH_ERR_ARG, "bad targets");
  std::vector<int32_t> nc((size_t)nt);
  for (int64_t q = 0; q < nt; ++q) {
    if (targets[q] < 0 || targets[q] >= c->n) return fail(c, SPH_ERR_ARG, "target %lld out of range", (long long)targets[q]);
    rc = cuda_check(c, cudaMemcpyAsync(&nc[q], c->nc + targets[q], 4, cudaMemcpyDeviceToHost, c->st), "nc copy");
    if (rc) return rc;
  }
  if ((rc = cuda_check(c, cudaStreamSynchronize(c->st), "sync"))) return rc;
  offsets[0] = 0;
  for (int64_t q = 0; q < nt; ++q) offsets[q + 1] = offsets[q] + std::min(nc[q], c->cfg.ngmax);
  if (offsets[nt] > idx_cap || (!idx && offsets[nt] > 0))
    return fail(c, SPH_ERR_CAPACITY, "idx_cap %lld < %lld neighbours", (long long)idx_cap, (long long)offsets[nt]);
  for (int64_t q = 0; q < nt; ++q) {
    const int64_t k = offsets[q + 1] - offsets[q];
    if (!k) continue;
    rc = cuda_check(c, cudaMemcpy2DAsync(idx + offsets[q], 4, c->nbr + targets[q], 4 * c->cfg.n_capacity, 4, k,
                                         cudaMemcpyDeviceToHost, c->st), "row copy");
    if (rc) return rc;
  }
  return cuda_check(c, cudaStreamSynchronize(c->st), "sync");
}

int sph_density(sph_ctx* c) {
  int rc = check_ready(c, S_NBR, "sph_density");
  return rc ? rc : body_simple(c, SPH_PHASE_DENSITY, S_DENS);
}

int sph_eos(sph_ctx* c) {
  int rc = check_ready(c, S_DENS, "sph_eos");
  if (rc) return rc;
  if (c->P.part == SPH_PART_GHOSTS) {  // the ghosts' EOS after their rho arrived: stage unchanged
    if (c->stage < S_EOS) return fail(c, SPH_ERR_STATE, "sph_eos(GHOSTS) needs a full sph_eos first");
    const int stage = c->stage;
    const bool gd = c->gradh_done;
    rc = body_simple(c, SPH_PHASE_EOS, stage);
    c->gradh_done = gd;
    return rc;
  }
  return body_simple(c, SPH_PHASE_EOS, S_EOS);
}

int sph_set_part(sph_ctx* c, int part) {
  int rc = check_ready(c, S_INIT, "sph_set_part");
  if (rc) return rc;
  if (part < SPH_PART_ALL || part > SPH_PART_GHOSTS) return fail(c, SPH_ERR_ARG, "unknown part %d", part);
  if (part != SPH_PART_ALL && (c->cfg.gradh || c->cfg.ve))
    return fail(c, SPH_ERR_NOT_SUPPORTED, "split IAD / momentum with grad-h or volume elements");
  c->P.part = part;
  return SPH_OK;
}

int sph_gradh(sph_ctx* c) {
  int rc = check_ready(c, S_EOS, "sph_gradh");
  if (rc) return rc;
  if (!c->cfg.gradh && !c->cfg.ve) return fail(c, SPH_ERR_STATE, "gradh not enabled (cfg.gradh = cfg.ve = 0)");
  return body_simple(c, SPH_PHASE_GRADH, S_EOS);
}

int sph_iad(sph_ctx* c) {
  int rc = check_ready(c, S_EOS, "sph_iad");
  if (rc) return rc;
  if ((c->cfg.gradh || c->cfg.ve) && !c->gradh_done)
    return fail(c, SPH_ERR_STATE, "cfg.gradh / cfg.ve: sph_gradh must run before sph_iad");
  if (c->P.part == SPH_PART_GHOSTS) return fail(c, SPH_ERR_ARG, "part GHOSTS is for sph_eos");
  // the INTERIOR half of a split IAD leaves the stage: the BOUNDARY half follows
  return body_simple(c, SPH_PHASE_IAD, c->P.part == SPH_PART_INTERIOR ? S_EOS : S_IAD);
}

int sph_momentum_energy(sph_ctx* c) {
  int rc = check_ready(c, S_IAD, "sph_momentum_energy");
  if (rc) return rc;
  if (c->P.part == SPH_PART_GHOSTS) return fail(c, SPH_ERR_ARG, "part GHOSTS is for sph_eos");
  return body_simple(c, SPH_PHASE_MOMENTUM_ENERGY, c->P.part == SPH_PART_INTERIOR ? S_IAD : S_MOM);
}

int sph_timestep(sph_ctx* c, double* dt) {
  int rc = check_ready(c, S_MOM, "sph_timestep");
  if (rc) return rc;
  if ((rc = body_simple(c, SPH_PHASE_TIMESTEP, S_DT))) return rc;
  rc = sync_scalars(c);
  if (dt) *dt = c->h_ds.dt;
  return rc;
}

int sph_update(sph_ctx* c) {
  int rc = check_ready(c, S_DT, "sph_update");
  return rc ? rc : body_simple(c, SPH_PHASE_UPDATE, S_PART);
}

static int sph_step_all(sph_ctx* c, sph_step_info* info);
int sph_step(sph_ctx* c, sph_step_info* info) {
  if (!c) return fail(nullptr, SPH_ERR_ARG, "sph_step: null context");
  const int part = c->P.part;  // a whole step is never split
  c->P.part = SPH_PART_ALL;
  const int rc_step = sph_step_all(c, info);
  c->P.part = part;
  return rc_step;
}

// The phases of one step, enqueued (no synchronisation).
static int step_body(sph_ctx* c) {
  int rc;
  if ((rc = body_tree(c))) return rc;
  if ((rc = body_neighbors(c))) return rc;
  if ((rc = body_simple(c, SPH_PHASE_DENSITY, S_DENS))) return rc;
  if ((rc = body_simple(c, SPH_PHASE_EOS, S_EOS))) return rc;
  if ((c->cfg.gradh || c->cfg.ve) && (rc = body_simple(c, SPH_PHASE_GRADH, S_EOS))) return rc;
  if ((rc = body_simple(c, SPH_PHASE_IAD, S_IAD))) return rc;
  if ((rc = body_simple(c, SPH_PHASE_MOMENTUM_ENERGY, S_MOM))) return rc;
  if (c->cfg.gravity && (rc = body_simple(c, SPH_PHASE_GRAVITY, S_MOM))) return rc;
  if (c->stir_on && (rc = body_simple(c, SPH_PHASE_STIR, S_MOM))) return rc;
  if ((rc = body_simple(c, SPH_PHASE_TIMESTEP, S_DT))) return rc;
  return body_simple(c, SPH_PHASE_UPDATE, S_PART);
}

// sph_step through a CUDA graph when nothing in the step needs the host between
// phases (no PHASE accounting, DVFS trace or clock policy): the ~22 launches
// and events of a step go to the device as one graph launch, so the short
// phases after the step's synchronisation do not wait on host enqueue.  The
// graph of a (buffer parity, sort passes, n) is captured from the eager body
// once; a replay re-applies the host-side state changes recorded then.
static bool graph_ok(const sph_ctx* c) {
  return !c->graphs_off && !c->acct.active && !c->trace.active && c->clock_mode == SPH_CLOCK_DEFAULT &&
         c->P.part == SPH_PART_ALL && !c->rec_m_dirty && c->n > 0;
}

static int step_graph(sph_ctx* c, bool* used) {
  *used = false;
  sph_ctx::StepGraph* g = nullptr;
  for (auto& x : c->graphs)
    if (x.valid && x.cur == c->cur && x.skip == c->sort_skip && x.n == c->n && x.stir_on == c->stir_on &&
        !memcmp(&x.P, &c->P, sizeof(Params)) && !memcmp(&x.stir, &c->stir, sizeof(Stir)))
      g = &x;
  if (g) {
    cudaError_t e = cudaGraphLaunch(g->exec, c->st);
    if (e != cudaSuccess) return cuda_check(c, e, "cudaGraphLaunch");
    c->cur = g->cur_after;
    c->last_perm = g->last_perm;
    c->key_sorted = g->key_sorted;
    c->inv_valid = false;
    c->gradh_done = g->gradh_done;
    for (int p = 0; p < SPH_NPHASES; ++p)
      if (g->ran[p]) {
        c->pending[p] = true;
        c->rows[p].calls++;
        c->rows[p].locked = 0;
      }
    note_launch((int)g->launches);
    c->stage = S_PART;
    *used = true;
    return SPH_OK;
  }
  // capture: the eager body enqueues into the capturing stream (nothing runs)
  const int cur0 = c->cur, skip0 = c->sort_skip;
  uint32_t* perm0 = c->last_perm;
  uint64_t* ks0 = c->key_sorted;
  const bool inv0 = c->inv_valid, gd0 = c->gradh_done;
  const int stage0 = c->stage;
  bool pend0[SPH_NPHASES];
  int64_t calls0[SPH_NPHASES];
  for (int p = 0; p < SPH_NPHASES; ++p) pend0[p] = c->pending[p], calls0[p] = c->rows[p].calls;
  const long long l0 = g_launches.load();
  auto restore = [&]() {
    c->cur = cur0;
    c->last_perm = perm0;
    c->key_sorted = ks0;
    c->inv_valid = inv0;
    c->gradh_done = gd0;
    c->stage = stage0;
    for (int p = 0; p < SPH_NPHASES; ++p) c->pending[p] = pend0[p], c->rows[p].calls = calls0[p];
    c->poisoned = false;
    c->err[0] = 0;
    cudaGetLastError();
    c->graphs_off = true;  // run eagerly from now on
  };
  if (cudaStreamBeginCapture(c->st, cudaStreamCaptureModeRelaxed) != cudaSuccess) {
    restore();
    return SPH_OK;
  }
  const int rc_body = step_body(c);
  cudaGraph_t graph = nullptr;
  const cudaError_t e_end = cudaStreamEndCapture(c->st, &graph);
  cudaGraphExec_t exec = nullptr;
  if (rc_body || e_end != cudaSuccess || !graph ||
      cudaGraphInstantiate(&exec, graph, 0) != cudaSuccess) {
    if (graph) cudaGraphDestroy(graph);
    restore();
    return SPH_OK;
  }
  cudaGraphDestroy(graph);
  g = &c->graphs[c->graph_next];
  c->graph_next = (c->graph_next + 1) % 4;
  if (g->exec) cudaGraphExecDestroy(g->exec);
  g->valid = true;
  g->cur = cur0;
  g->skip = skip0;
  g->n = c->n;
  g->P = c->P;
  g->stir = c->stir;
  g->stir_on = c->stir_on;
  g->exec = exec;
  g->cur_after = c->cur;
  g->last_perm = c->last_perm;
  g->key_sorted = c->key_sorted;
  g->gradh_done = c->gradh_done;
  for (int p = 0; p < SPH_NPHASES; ++p) g->ran[p] = c->rows[p].calls != calls0[p];
  g->launches = g_launches.load() - l0;
  const cudaError_t e = cudaGraphLaunch(exec, c->st);
  if (e != cudaSuccess) return cuda_check(c, e, "cudaGraphLaunch");
  *used = true;
  return SPH_OK;
}

static int sph_step_all(sph_ctx* c, sph_step_info* info) {
  int rc = check_ready(c, S_PART, "sph_step");
  if (rc) return rc;
  bool used = false;
  if (graph_ok(c) && (rc = step_graph(c, &used))) return rc;
  // A data error (capacity, singular, box) makes the update meaningless: check
  // the device status after the update is enqueued (one sync per step).
  if (!used && (rc = step_body(c))) return rc;
  rc = sync_scalars(c);
  if (info) {
    info->t = c->h_ds.t;
    info->dt = c->h_ds.dt;
    fill_stats(c, &info->nbr);
    info->cell_level = c->h_ds.cell_level;
    info->graph = used ? 1 : 0;
    for (int p = 0; p < SPH_NPHASES; ++p) info->phase_ms[p] = c->last_ms[p];
    info->grav_multipoles = (int64_t)c->h_ds.grav_mp;
    info->grav_pairs = (int64_t)c->h_ds.grav_pp;
    info->grav_pops = (int64_t)c->h_ds.grav_pops;
  }
  return rc;
}

int sph_set_clock_policy(sph_ctx* c, int mode, const uint32_t mhz[SPH_NPHASES]) {
  int rc = check_ready(c, S_INIT, "sph_set_clock_policy");
  if (rc) return rc;
  if (mode == SPH_CLOCK_DEFAULT) {
    if (c->locked_any) c->nvml.reset_sm_clock();
    c->locked_any = false;
    c->current_lock = 0;
    c->clock_mode = SPH_CLOCK_DEFAULT;
    for (int p = 0; p < SPH_NPHASES; ++p) c->clock_mhz[p] = 0;
    return SPH_OK;
  }
  if (mode != SPH_CLOCK_STATIC && mode != SPH_CLOCK_PER_PHASE) return fail(c, SPH_ERR_ARG, "unknown clock mode %d", mode);
  if (!mhz) return fail(c, SPH_ERR_ARG, "null mhz");
  const char* allow = getenv("SPH_ALLOW_CLOCK_CONTROL");
  if (!allow || strcmp(allow, "1") != 0)
    return fail(c, SPH_ERR_NO_PERMISSION, "clock control disabled: this host forbids clock changes (set SPH_ALLOW_CLOCK_CONTROL=1 where locking SM clocks is permitted)");
  if (!c->nvml.ok) return fail(c, SPH_ERR_NOT_SUPPORTED, "NVML unavailable: %s", c->nvml.err);
  unsigned sup[512];
  int ns = c->nvml.supported_sm_clocks(sup, 512);
  if (ns <= 0) return fail(c, SPH_ERR_NOT_SUPPORTED, "no supported graphics clocks reported");
  unsigned want[SPH_NPHASES];
  for (int p = 0; p < SPH_NPHASES; ++p) {
    unsigned r = mode == SPH_CLOCK_STATIC ? mhz[0] : mhz[p];
    if (r == 0) { want[p] = 0; continue; }
    unsigned best = sup[0];
    for (int k = 1; k < ns; ++k)
      if ((sup[k] > r ? sup[k] - r : r - sup[k]) < (best > r ? best - r : r - best)) best = sup[k];
    want[p] = best;
  }
  unsigned probe = 0;
  for (int p = 0; p < SPH_NPHASES; ++p) if (want[p]) { probe = want[p]; break; }
  if (probe) {
    int lrc = c->nvml.lock_sm_clock(probe);
    if (lrc == 4) return fail(c, SPH_ERR_NO_PERMISSION, "nvmlDeviceSetGpuLockedClocks: no permission");
    if (lrc != 0) return fail(c, SPH_ERR_NOT_SUPPORTED, "nvmlDeviceSetGpuLockedClocks: %s", c->nvml.error_string(lrc));
    c->locked_any = true;
    c->current_lock = probe;
  }
  for (int p = 0; p < SPH_NPHASES; ++p) c->clock_mhz[p] = want[p];
  c->clock_mode = mode;
  return SPH_OK;
}

int sph_energy_report(sph_ctx* c, sph_energy_row* rows, int cap, int* n_rows) {
  int rc = check_ready(c, S_INIT, "sph_energy_report");
  if (rc) return rc;
  if (!rows || cap < SPH_NPHASES) return fail(c, SPH_ERR_ARG, "need room for %d rows", SPH_NPHASES);
  if (!c->poisoned) {
    rc = cuda_check(c, cudaStreamSynchronize(c->st), "sync");
    if (rc) return rc;
    collect_all(c);
  }
  for (int p = 0; p < SPH_NPHASES; ++p) {
    sph_energy_row& r = rows[p];
    memset(&r, 0, sizeof(r));
    r.phase = p;
    snprintf(r.name, sizeof(r.name), "%s", kPhaseNames[p]);
    r.calls = c->rows[p].calls;
    r.seconds = c->rows[p].seconds;
    {
      std::lock_guard<std::mutex> g(c->acct.mu);
      r.joules = c->acct.J[p];
      r.mean_sm_mhz = c->acct.mhz_n[p] ? c->acct.mhz_sum[p] / c->acct.mhz_n[p] : 0.0;
      r.available = c->acct.samples > 0 ? 1 : 0;
    }
    r.locked_mhz = c->rows[p].locked;
  }
  if (n_rows) *n_rows = SPH_NPHASES;
  return SPH_OK;
}

int sph_energy_reset(sph_ctx* c) {
  int rc = check_ready(c, S_INIT, "sph_energy_reset");
  if (rc) return rc;
  cudaStreamSynchronize(c->st);
  collect_all(c);
  for (int p = 0; p < SPH_NPHASES; ++p) c->rows[p] = PhaseRow();
  acct_reset(c);
  return SPH_OK;
}

int sph_energy_totals(sph_ctx* c, sph_energy_window* t) {
  int rc = check_ready(c, S_INIT, "sph_energy_totals");
  if (rc) return rc;
  if (!t) return fail(c, SPH_ERR_ARG, "null totals");
  if (!c->poisoned && (rc = cuda_check(c, cudaStreamSynchronize(c->st), "sync"))) return rc;
  memset(t, 0, sizeof(*t));
  unsigned long long e1 = 0;
  const bool eok = c->nvml.energy_mj(&e1);
  std::lock_guard<std::mutex> g(c->acct.mu);
  t->wall_seconds = std::chrono::duration<double>(std::chrono::steady_clock::now() - c->acct.t_start).count();
  t->sampled_seconds = c->acct.seconds;
  for (int p = 0; p <= SPH_NPHASES; ++p) t->sampled_joules += c->acct.J[p];
  t->between_joules = c->acct.J[SPH_NPHASES];
  t->counter_joules = (eok && c->acct.e_start_ok) ? (double)(e1 - c->acct.e_start) * 1e-3 : -1.0;
  t->samples = c->acct.samples;
  return SPH_OK;
}

int sph_energy_counter_mj(sph_ctx* c, uint64_t* mj) {
  if (!c || !mj) return fail(nullptr, SPH_ERR_ARG, "null argument");
  unsigned long long v;
  if (!c->nvml.energy_mj(&v)) return fail(c, SPH_ERR_NVML, "NVML energy counter unavailable: %s", c->nvml.err);
  *mj = v;
  return SPH_OK;
}

int sph_set_accounting(sph_ctx* c, int mode) {
  int rc = check_ready(c, S_INIT, "sph_set_accounting");
  if (rc) return rc;
  if (mode != SPH_ACCOUNTING_OFF && mode != SPH_ACCOUNTING_PHASE) return fail(c, SPH_ERR_ARG, "unknown accounting mode %d", mode);
  if (mode == SPH_ACCOUNTING_PHASE) {
    if ((rc = acct_start(c))) return rc;
  } else {
    acct_stop(c);
  }
  c->cfg.accounting = mode;
  return SPH_OK;
}

int sph_kernel_launches(int64_t* count) {
  if (!count) return fail(nullptr, SPH_ERR_ARG, "null count");
  *count = (int64_t)g_launches.load();
  return SPH_OK;
}

int sph_repeat_phase(sph_ctx* c, int phase, int reps, double* ms_per_call, double* joules_per_call) {
  int need;
  switch (phase) {
    case SPH_PHASE_KEYS: need = S_TREE; break;
    case SPH_PHASE_SORT: need = S_TREE; break;
    case SPH_PHASE_CELLS: need = S_TREE; break;
    case SPH_PHASE_NEIGHBORS: need = S_TREE; break;
    case SPH_PHASE_DENSITY:
      // after the volume-element GRADH, DENSITY would overwrite the normalised rho
      // with rho0 (reading 23): not repeatable without re-running GRADH
      if (c && c->cfg.ve && c->gradh_done)
        return fail(c, SPH_ERR_STATE, "DENSITY is not repeatable after the volume-element GRADH");
      need = S_NBR;
      break;
    case SPH_PHASE_EOS: need = S_DENS; break;
    case SPH_PHASE_IAD: need = S_EOS; break;
    case SPH_PHASE_GRADH:
      // (with cfg.ve the phase rewrites rho from itself: not repeatable)
      if (!c || !c->cfg.gradh || c->cfg.ve) return fail(c, SPH_ERR_STATE, "GRADH repeatable only with cfg.gradh and no cfg.ve");
      need = S_EOS;
      break;
    case SPH_PHASE_MOMENTUM_ENERGY: need = S_IAD; break;
    case SPH_PHASE_TIMESTEP: need = S_DT; break;
    default: return fail(c, SPH_ERR_ARG, "phase %d is not repeatable (it changes the state)", phase);
  }
  int rc = check_ready(c, need, "sph_repeat_phase");
  if (rc) return rc;
  if (reps < 1) return fail(c, SPH_ERR_ARG, "reps < 1");
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  rc = cuda_check(c, cudaStreamSynchronize(c->st), "sync");
  if (rc) return rc;
  apply_clock(c, phase);
  unsigned long long e0 = 0, e1 = 0;
  bool eok = c->nvml.energy_mj(&e0);
  cudaEventRecord(a, c->st);
  Fields F = fields(c);
  Params Pr = c->P;  // whole phases (not a split half)
  Pr.part = SPH_PART_ALL;
  // KEYS writes into the key buffer not holding the sorted keys; SORT re-sorts
  // the (already sorted) keys in place and permutes into the spare state buffer
  // without switching to it: both leave the pipeline state unchanged.
  uint64_t* spare_keys = c->key_sorted == c->keyA ? c->keyB : c->keyA;
  Fields Fk = F;
  Fk.key = spare_keys;
  const int prv = c->cur;
  const size_t perm_bytes = sizeof(uint32_t) * (size_t)c->n;
  if (phase == SPH_PHASE_SORT && c->last_perm && c->n > 0) {  // the repeats reuse its buffer
    cudaMemcpyAsync(c->perm_saved, c->last_perm, perm_bytes, cudaMemcpyDeviceToDevice, c->st);
    c->inv_valid = false;
  }
  // EOS after GRADH: p/(Omega rho^2), as the pipeline left it (reading 21)
  const bool eos_omega = c->gradh_done && c->cfg.gradh;
  for (int r = 0; r < reps; ++r) {
    switch (phase) {
      case SPH_PHASE_KEYS: launch_box_keys(Fk, Pr, c->st); break;
      case SPH_PHASE_SORT: {
        uint32_t* perm = nullptr;
        uint64_t* ks = nullptr;
        launch_sort(F, c->key_sorted, spare_keys, c->valA, c->valB, c->sort_hist, c->sort_status,
                    c->status_bytes, &perm, &ks, c->st, c->sort_skip);
        c->cur = prv ^ 1;
        Fields Fd = fields(c);
        c->cur = prv;
        launch_permute(Fd, perm, c->state[prv], c->ids[prv], c->st);
        break;
      }
      case SPH_PHASE_CELLS: launch_cells(F, Pr, c->level_cap, c->st); break;
      case SPH_PHASE_TIMESTEP: launch_timestep(F, Pr, c->st); break;
      case SPH_PHASE_NEIGHBORS: launch_neighbors(F, Pr, c->st); break;
      case SPH_PHASE_DENSITY: launch_density(F, Pr, c->st); break;
      case SPH_PHASE_EOS: launch_eos(F, Pr, c->st, eos_omega); break;
      case SPH_PHASE_IAD: launch_iad(F, Pr, c->st); break;
      case SPH_PHASE_GRADH: launch_gradh(F, Pr, c->st); break;
      case SPH_PHASE_MOMENTUM_ENERGY: launch_momentum_energy(F, Pr, c->st); break;
    }
  }
  cudaEventRecord(b, c->st);
  if (phase == SPH_PHASE_SORT && c->last_perm && c->n > 0)
    cudaMemcpyAsync(c->last_perm, c->perm_saved, perm_bytes, cudaMemcpyDeviceToDevice, c->st);
  rc = cuda_check(c, cudaEventSynchronize(b), "repeat");
  if (!rc) {
    eok = eok && c->nvml.energy_mj(&e1);
    float ms = 0;
    cudaEventElapsedTime(&ms, a, b);
    if (ms_per_call) *ms_per_call = ms / reps;
    if (joules_per_call) *joules_per_call = eok ? (double)(e1 - e0) * 1e-3 / reps : -1.0;
  }
  cudaEventDestroy(a);
  cudaEventDestroy(b);
  return rc;
}

}  // extern "C"

// ------------------------------------------------------------------ DVFS trace
int sph_trace_start(sph_ctx* c, double period_ms, int64_t capacity) {
  int rc = check_ready(c, S_INIT, "sph_trace_start");
  if (rc) return rc;
  if (!(period_ms >= 0.1) || capacity < 1) return fail(c, SPH_ERR_ARG, "period_ms >= 0.1 and capacity >= 1 required");
  if (c->trace.active) return fail(c, SPH_ERR_STATE, "a trace is already running");
  if (!c->nvml.ok) return fail(c, SPH_ERR_NVML, "NVML unavailable: %s", c->nvml.err);
  if ((rc = ensure_phase_word(c))) return rc;
  if (!c->acct.active) *c->trace.word = -1;
  c->trace.buf.assign((size_t)capacity, sph_trace_sample{});
  c->trace.taken = 0;
  c->trace.run.store(true);
  c->trace.active = true;
  sph_ctx::Trace* T = &c->trace;
  Nvml* nv = &c->nvml;
  c->trace.th = std::thread([T, nv, period_ms]() {
    using clk = std::chrono::steady_clock;
    const auto t0 = clk::now();
    const auto dt = std::chrono::duration_cast<clk::duration>(std::chrono::duration<double, std::milli>(period_ms));
    auto next = t0;
    while (T->run.load(std::memory_order_relaxed)) {
      sph_trace_sample s{};
      const auto q0 = clk::now();
      s.t_ms = std::chrono::duration<double, std::milli>(q0 - t0).count();
      s.phase = *T->word;
      unsigned v = 0;
      if (nv->sm_clock_mhz(&v)) s.sm_mhz = v;
      if (nv->power_mw(&v)) s.power_mw = v;
      unsigned long long e = 0;
      if (nv->energy_mj(&e)) s.energy_mj = e;
      s.query_us = (uint32_t)std::chrono::duration<double, std::micro>(clk::now() - q0).count();
      if (T->taken < (int64_t)T->buf.size()) T->buf[(size_t)T->taken] = s;
      ++T->taken;
      next += dt;
      const auto now = clk::now();
      if (next < now) next = now;
      std::this_thread::sleep_until(next);
    }
  });
  return SPH_OK;
}

int sph_trace_stop(sph_ctx* c, sph_trace_sample* out, int64_t cap, int64_t* n) {
  if (!c) return fail(nullptr, SPH_ERR_ARG, "sph_trace_stop: null context");
  if (!c->trace.active) return fail(c, SPH_ERR_STATE, "no trace running");
  if (cap < 0 || (cap > 0 && !out)) return fail(c, SPH_ERR_ARG, "bad output buffer");
  c->trace.run.store(false);
  if (c->trace.th.joinable()) c->trace.th.join();
  c->trace.active = false;
  const int64_t m = std::min<int64_t>(std::min<int64_t>(c->trace.taken, (int64_t)c->trace.buf.size()), cap);
  for (int64_t k = 0; k < m; ++k) out[k] = c->trace.buf[(size_t)k];
  if (n) *n = c->trace.taken;
  return SPH_OK;
}

// ------------------------------------------------------------------ driving
int sph_stir_modes(int32_t* n3, int cap) {
  if (!n3 || cap < kStirModes) return -SPH_ERR_ARG;
  return stir_modes(n3);
}

int sph_stir_init(sph_ctx* c, const sph_stir_params* prm, const double* w, const double* A0,
                  const double* noise, int64_t nsteps, int mem) {
  int rc = check_ready(c, S_INIT, "sph_stir_init");
  if (rc) return rc;
  if (c->cfg.stir_steps == 0) return fail(c, SPH_ERR_NOT_SUPPORTED, "driving needs cfg.stir_steps > 0 (arena room for the noise table)");
  if (!c->cfg.periodic[0] || !c->cfg.periodic[1] || !c->cfg.periodic[2])
    return fail(c, SPH_ERR_NOT_SUPPORTED, "driving is defined on a fully periodic box");
  if (!prm || !w || !noise) return fail(c, SPH_ERR_ARG, "null params, weights or noise");
  if (nsteps < 1 || nsteps > c->cfg.stir_steps) return fail(c, SPH_ERR_ARG, "nsteps must be in [1, stir_steps = %d]", c->cfg.stir_steps);
  if (!(prm->t_decay > 0) || !(prm->sigma >= 0) || !(prm->sol_weight >= 0 && prm->sol_weight <= 1))
    return fail(c, SPH_ERR_ARG, "need t_decay > 0, sigma >= 0, 0 <= sol_weight <= 1");
  if (mem != SPH_MEM_HOST && mem != SPH_MEM_DEVICE) return fail(c, SPH_ERR_ARG, "mem must be HOST or DEVICE");
  stir_upload_modes();
  const cudaMemcpyKind k = mem == SPH_MEM_HOST ? cudaMemcpyHostToDevice : cudaMemcpyDeviceToDevice;
  const size_t M6 = sizeof(double) * kStirModes * 6;
  rc = cuda_check(c, cudaMemcpyAsync(c->stir.w, w, sizeof(double) * kStirModes, k, c->st), "stir w");
  if (!rc) rc = cuda_check(c, A0 ? cudaMemcpyAsync(c->stir.A, A0, M6, k, c->st) : cudaMemsetAsync(c->stir.A, 0, M6, c->st), "stir A0");
  if (!rc) rc = cuda_check(c, cudaMemcpyAsync(c->stir.noise, noise, M6 * (size_t)nsteps, k, c->st), "stir noise");
  if (!rc) rc = cuda_check(c, cudaMemsetAsync(&c->ds->stir_step, 0, sizeof(unsigned long long), c->st), "stir counter");
  if (!rc) rc = cuda_check(c, cudaStreamSynchronize(c->st), "sync");
  if (rc) return rc;
  c->stir.nsteps = nsteps;
  c->stir.sigma = prm->sigma;
  c->stir.t_decay = prm->t_decay;
  c->stir.zeta = prm->sol_weight;
  c->stir_on = true;
  return SPH_OK;
}

int sph_stir(sph_ctx* c) {
  int rc = check_ready(c, S_MOM, "sph_stir");
  if (rc) return rc;
  if (!c->stir_on) return fail(c, SPH_ERR_STATE, "driving not enabled (sph_stir_init)");
  return body_simple(c, SPH_PHASE_STIR, S_MOM);
}

int sph_stir_get_state(sph_ctx* c, double* A, int64_t* steps) {
  int rc = check_ready(c, S_INIT, "sph_stir_get_state");
  if (rc) return rc;
  if (!c->stir_on) return fail(c, SPH_ERR_STATE, "driving not enabled (sph_stir_init)");
  if (A) rc = cuda_check(c, cudaMemcpyAsync(A, c->stir.A, sizeof(double) * kStirModes * 6, cudaMemcpyDeviceToHost, c->st), "stir A");
  if (rc) return rc;
  rc = sync_scalars(c);
  if (steps) *steps = (int64_t)c->h_ds.stir_step;
  return rc;
}

int sph_supported_clocks(sph_ctx* c, uint32_t* mhz, int cap, int* n) {
  int rc = check_ready(c, S_INIT, "sph_supported_clocks");
  if (rc) return rc;
  if (!mhz || cap < 1 || !n) return fail(c, SPH_ERR_ARG, "bad output buffer");
  if (!c->nvml.ok) return fail(c, SPH_ERR_NVML, "NVML unavailable: %s", c->nvml.err);
  unsigned sup[512];
  int ns = c->nvml.supported_sm_clocks(sup, 512);
  if (ns <= 0) return fail(c, SPH_ERR_NVML, "no supported graphics clocks reported");
  std::sort(sup, sup + ns, [](unsigned a, unsigned b) { return a > b; });
  *n = std::min(ns, cap);
  for (int k = 0; k < *n; ++k) mhz[k] = sup[k];
  return SPH_OK;
}

int sph_gravity(sph_ctx* c) {
  int rc = check_ready(c, S_MOM, "sph_gravity");
  if (rc) return rc;
  if (!c->cfg.gravity) return fail(c, SPH_ERR_STATE, "gravity not enabled (cfg.gravity = 0)");
  return body_simple(c, SPH_PHASE_GRAVITY, S_MOM);
}
