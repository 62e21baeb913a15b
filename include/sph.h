/*
 * sph.h -- C ABI of libsph, the B200-native SPH time-step library.
 *
 * What it computes.  One SPH-EXA hydro time step as measured by Simsek,
 * Piccinali and Ciorba (SC'24 workshops, /root/reference/PAPER.md, "P:NN" =
 * line NN): the particle keys of DomainDecompAndSync, neighbour
 * search, XMass / density, equation of state, IADVelocityDivCurl
 * (matrix part), MomentumEnergy, the end-of-step
 * time-step collective and the update -- each wrapped by the
 * per-function energy hooks of P:69-73 and, optionally, the per-function SM
 * clock of P:73.  PAPER.md prints no SPH formula; the formulas are
 * the readings of SURVEY.md 8(c) "Algorithm, step by step" (items 1-10),
 * restated in DESIGN.md section 3.  Each entry point below cites its item.
 *
 * Conventions (apply to every function):
 *  - Return value: SPH_OK (0) or one of the sph_status codes.  The message of
 *    the last error is sph_last_error(ctx).  No C++ exception or abort crosses
 *    this boundary.
 *  - Argument errors (SPH_ERR_ARG) leave the context unchanged.
 *  - CUDA errors are sticky: the context is poisoned and every later call
 *    returns SPH_ERR_STATE until sph_finalize.
 *  - Data errors detected on the device (degenerate open box, neighbour
 *    capacity exceeded, singular IAD matrix) are reported at the next call that
 *    synchronises (sph_find_neighbors, sph_timestep, sph_step, sph_get_*), do
 *    not poison, and leave the outputs of the failing phase unspecified.
 *  - NVML errors never poison: energy rows are marked unavailable, a refused
 *    clock policy reverts to SPH_CLOCK_DEFAULT.
 *  - Ownership: the caller owns ALL device memory (one byte arena of at least
 *    sph_workspace_size bytes, 256-byte aligned, that must outlive the context)
 *    and the CUDA stream.  The library sub-allocates fields, double buffers and
 *    scratch inside the arena and allocates nothing on the device itself.  It
 *    owns only its NVML handle and small host bookkeeping.
 *  - Work is enqueued asynchronously on the caller's stream.  Calls that return
 *    host values (sph_find_neighbors stats, sph_timestep, sph_step, sph_get_*,
 *    accounting phase edges) synchronise that stream.
 *  - One context per device per thread; a context is not internally
 *    thread-safe.
 *  - Particle arrays are fp64 structure-of-arrays; after sph_build_tree the
 *    particles are held in Morton (SFC) order and every per-particle output is
 *    in that order (SPH_F_ID gives the original ids).
 */
#ifndef SPH_H
#define SPH_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define SPH_ABI_VERSION 1

typedef enum sph_status {
  SPH_OK = 0,
  SPH_ERR_ARG = 1,           /* invalid argument; nothing changed            */
  SPH_ERR_STATE = 2,         /* call out of order, or context poisoned       */
  SPH_ERR_CUDA = 3,          /* CUDA runtime error (poisons the context)     */
  SPH_ERR_NCCL = 4,          /* reserved: multi-GPU communicator error        */
  SPH_ERR_NVML = 5,          /* NVML unavailable or failed (never poisons)   */
  SPH_ERR_NO_PERMISSION = 6, /* clock control refused by the host            */
  SPH_ERR_NOT_SUPPORTED = 7, /* feature not supported on this device/host   */
  SPH_ERR_CAPACITY = 8,      /* n > n_capacity or neighbour count > ngmax    */
  SPH_ERR_HCAP = 9,          /* reserved                                      */
  SPH_ERR_SINGULAR = 10,     /* IAD matrix with det <= 0 or non-finite       */
  SPH_ERR_BOX = 11           /* open axis with max == min                    */
} sph_status;

typedef enum sph_eos_kind { SPH_EOS_IDEAL = 0, SPH_EOS_ISOTHERMAL = 1 } sph_eos_kind;
typedef enum sph_mem_kind {
  SPH_MEM_HOST = 0,       /* host memory; the call synchronises                      */
  SPH_MEM_DEVICE = 1,     /* device memory; asynchronous on the context's stream     */
  SPH_MEM_HOST_ASYNC = 2  /* sph_get_field only: asynchronous copy into (pinned) host
                             memory, valid after sph_sync -- lets a caller overlap a
                             step's read-back with other work                        */
} sph_mem_kind;
typedef enum sph_accounting_mode {
  SPH_ACCOUNTING_OFF = 0,   /* CUDA-event phase times only, no phase-edge syncs  */
  SPH_ACCOUNTING_PHASE = 1  /* + in-situ energy per phase ("from the start of
                               each function call until its completion"): a host
                               thread samples the phase the device runs (written
                               by a 1-thread kernel at every phase edge) and the
                               NVML instant power every ~0.25 ms and integrates
                               P dt per phase.  No phase-edge syncs.  The B200
                               refreshes that power value every ~100 ms, so a
                               phase's joules are its device time at the power
                               around it; isolated per-phase power needs
                               sph_repeat_phase (REPEAT analog)          */
} sph_accounting_mode;

/* Phases = the functions whose energy the paper measures (Fig. 5).
 * DomainDecompAndSync = KEYS + SORT + CELLS on one GPU. */
typedef enum sph_phase {
  SPH_PHASE_KEYS = 0,            /* box reduction + 63-bit Morton keys (item 1-2) */
  SPH_PHASE_SORT = 1,            /* radix sort + permutation of all fields (3)    */
  SPH_PHASE_CELLS = 2,           /* cell table over the sorted keys               */
  SPH_PHASE_NEIGHBORS = 3,       /* neighbour lists (item 4)                      */
  SPH_PHASE_DENSITY = 4,         /* XMass / density (item 5)                      */
  SPH_PHASE_EOS = 5,             /* equation of state (item 6)                    */
  SPH_PHASE_IAD = 6,             /* IAD matrices (item 7)                         */
  SPH_PHASE_MOMENTUM_ENERGY = 7, /* momentum + energy + AV, local dt min (item 8) */
  SPH_PHASE_TIMESTEP = 8,        /* global dt (item 9; the P:220 collective)      */
  SPH_PHASE_UPDATE = 9,          /* positions, velocities, energy, h (item 10)    */
  SPH_PHASE_STIR = 10,           /* turbulence driving; runs after
                                    MOMENTUM_ENERGY, before TIMESTEP, when enabled */
  SPH_PHASE_GRAVITY = 11,        /* self-gravity; runs after
                                    MOMENTUM_ENERGY when cfg.gravity              */
  SPH_PHASE_GRADH = 12,          /* NormalizationGradh (reading 21); runs
                                    after EOS, before IAD, when cfg.gradh          */
  SPH_NPHASES = 13
} sph_phase;

typedef enum sph_clock_mode {
  SPH_CLOCK_DEFAULT = 0,   /* driver DVFS (the paper's "DVFS" arm)            */
  SPH_CLOCK_STATIC = 1,    /* one locked SM clock for every phase        */
  SPH_CLOCK_PER_PHASE = 2  /* SM clock set before each phase ("ManDyn")   */
} sph_clock_mode;

/* Per-particle fields readable with sph_get_field (all in the current order). */
typedef enum sph_field {
  SPH_F_X = 0, SPH_F_Y, SPH_F_Z, SPH_F_VX, SPH_F_VY, SPH_F_VZ, SPH_F_H, SPH_F_M, SPH_F_U,
  SPH_F_DU_M1,
  SPH_F_ID,     /* int64: original particle id (the Morton order as an id list)   */
  SPH_F_KEY,    /* uint64: Morton key (valid after sph_build_tree)                */
  SPH_F_NC,     /* int32: neighbour count (valid after sph_find_neighbors)        */
  SPH_F_RHO, SPH_F_P, SPH_F_C,
  SPH_F_C11, SPH_F_C12, SPH_F_C13, SPH_F_C22, SPH_F_C23, SPH_F_C33,
  SPH_F_AX, SPH_F_AY, SPH_F_AZ, SPH_F_DU,
  SPH_F_DIVV,   /* velocity divergence (cfg.divcurl; valid after sph_iad)       */
  SPH_F_CURLX, SPH_F_CURLY, SPH_F_CURLZ,  /* velocity curl (cfg.divcurl)        */
  SPH_F_BAL,    /* Balsara switch factor (cfg.av_switch; valid after sph_iad)  */
  SPH_F_PHI,    /* gravitational potential (cfg.gravity; after sph_gravity)    */
  SPH_F_OMEGA,  /* grad-h factor Omega (cfg.gradh; valid after sph_gradh)        */
  SPH_F_VSIG,   /* signal velocity (cfg.dt_vsig; after sph_momentum_energy)    */
  SPH_F_ORDER,  /* int32: pre-sort index of each position (after sph_build_tree) */
  SPH_NFIELDS
} sph_field;

/* Step configuration.  Values are inputs to the method (SURVEY 8(c) parameter
 * table); sph_config_default fills the proposed defaults. */
typedef struct sph_config {
  int64_t n_capacity;       /* max particles held (< 2^30)                        */
  double box_min[3];        /* periodic axes: the fixed box; open axes: ignored   */
  double box_max[3];
  int32_t periodic[3];      /* 1 = periodic axis (minimum image + wrap)           */
  int32_t eos;              /* sph_eos_kind                                        */
  double gamma;             /* ideal-gas gamma                                     */
  double cs0;               /* isothermal sound speed                              */
  double K;                 /* sinc-kernel (n = 6) normalisation                   */
  double ng0;               /* target neighbour count of the h update              */
  int32_t ngmax;            /* neighbour-list capacity per particle (never truncates:
                               overflow -> SPH_ERR_CAPACITY)                       */
  int32_t max_cell_level;   /* finest cell-grid level L (8^L cells), in [1, 10]    */
  double h_cap;             /* h <= h_cap after the update (periodic: <= min L / 4) */
  double k_cour;            /* Courant factor                                      */
  double dt_max_growth;     /* dt <= growth * dt_prev                              */
  double dt_first;          /* dt_prev before the first step                       */
  double av_alpha, av_beta, av_eps;
  int32_t device;           /* CUDA device ordinal the arena lives on              */
  int32_t accounting;       /* sph_accounting_mode                                 */
  int32_t rank, nranks;     /* reserved for SFC domain decomposition (1 rank now)  */
  int32_t stir_steps;       /* capacity (steps) of the driving-noise table; 0 = no
                               turbulence driving (sph_stir_init)                  */
  int32_t divcurl;          /* 1: IADVelocityDivCurl also computes div v, curl v
                               (reading 19)                                        */
  int32_t av_switch;        /* 1: Balsara switch on the AV (implies divcurl)       */
  int32_t gravity;          /* 1: self-gravity phase (open boxes only)             */
  int32_t grav_level;       /* leaf level Lt of the gravity octree, 1..8           */
  double grav_G;            /* gravitational constant                              */
  double grav_eps;          /* Plummer softening length                            */
  double grav_theta;        /* opening angle: multipole when side < theta * dist;
                               0 = direct summation                               */
  int32_t gradh;            /* 1: NormalizationGradh phase; momentum-energy uses
                               p / (Omega rho^2) (reading 21)                     */
  int32_t dt_vsig;          /* 1: signal-velocity time step (reading 22) instead of
                               C min h/c                                          */
  int32_t ve;               /* 1: generalized volume elements X = m/rho0 (reading
                               23): GRADH normalises the density                  */
  int32_t grav_fp64;        /* gravity with theta > 0: 0 (default) evaluates each
                               multipole / direct term in fp32 from positions
                               relative to the walking group's centre and adds it
                               to fp64 accumulators (rounding ~1e-7 of a term,
                               far below the tree's truncation error); 1 = fp64
                               terms.  theta = 0 (the direct sum) is always fp64. */
  int32_t reserved[4];
} sph_config;

typedef struct sph_nbr_stats {
  int32_t min_nc, max_nc;   /* over all particles                                  */
  double mean_nc;
  int64_t total;            /* sum of nc                                           */
  int64_t candidates;       /* diagnostic: candidate tests of the search (per lane) */
  int64_t passes;           /* diagnostic: warp passes of the search               */
} sph_nbr_stats;

typedef struct sph_step_info {
  double t;                 /* simulation time after the step                      */
  double dt;                /* the step's dt                                       */
  sph_nbr_stats nbr;
  int32_t cell_level;       /* cell-grid level used by the neighbour search        */
  int32_t graph;            /* 1: the step's phases ran as one CUDA graph launch
                               (captured at the first step of a buffer parity /
                               sort pass count / n; env SPH_NO_GRAPH=1 disables) */
  double phase_ms[SPH_NPHASES]; /* CUDA-event time of each phase in this step      */
  int64_t grav_multipoles;  /* diagnostic: multipoles evaluated per warp, summed    */
  int64_t grav_pairs;       /* diagnostic: direct pairs per warp (32 targets), sum */
  int64_t grav_pops;        /* diagnostic: tree nodes opened per warp, summed      */
} sph_step_info;

typedef struct sph_energy_row {
  int32_t phase;            /* sph_phase                                           */
  char name[32];
  int64_t calls;
  double seconds;           /* accumulated CUDA-event time                         */
  double joules;            /* sampled energy while the device ran the phase (PHASE) */
  double mean_sm_mhz;       /* mean SM clock sampled while it ran (PHASE)          */
  uint32_t locked_mhz;      /* clock requested by the policy, 0 = default          */
  int32_t available;        /* 1 if joules are valid                               */
} sph_energy_row;

/* One sample of the DVFS trace (Fig. 9: the SM clock the driver
 * picks while each function runs, over a few time steps). */
typedef struct sph_trace_sample {
  double t_ms;              /* host steady-clock time since sph_trace_start      */
  int32_t phase;            /* sph_phase running on the device, -1 between phases */
  uint32_t sm_mhz;          /* nvmlDeviceGetClockInfo(NVML_CLOCK_SM)              */
  uint32_t power_mw;        /* nvmlDeviceGetPowerUsage                            */
  uint32_t query_us;        /* time the three NVML queries of this sample took    */
  uint64_t energy_mj;       /* nvmlDeviceGetTotalEnergyConsumption                */
} sph_trace_sample;

/* Turbulence driving (Ornstein-Uhlenbeck stirring of the
 * Subsonic Turbulence workload).  The mode set is fixed: the
 * SPH_STIR_NMODES integer wave vectors n with 1 <= |n|^2 <= 9 in the half space
 * (n_x > 0, or n_x = 0 and n_y > 0, or n_x = n_y = 0 and n_z > 0), in
 * lexicographic order of (n_x, n_y, n_z) (sph_stir_modes), k_a = 2 pi n_a / L_a.
 * Per mode the OU state holds a complex 3-vector A (6 doubles: Re x, Im x, Re y,
 * Im y, Re z, Im z).  One STIR phase (step s = number of phases run so far):
 *   A <- f A + sigma sqrt(1 - f^2) xi_s,  f = exp(-dt_prev / t_decay)
 *   (xi_s = row s of the caller's Gaussian noise table: the random numbers are
 *   inputs, so the oracle draws nothing);
 *   A^ = zeta P_perp A + (1 - zeta) P_par A  (P_perp = I - k^k^T, P_par = k^k^T);
 *   a_i += 2 sum_m w_m Re( A^_m exp(i k_m . (x_i - box_min)) ).
 * Weights w_m, sigma, t_decay and zeta are conventions (parity unpinned). */
#define SPH_STIR_NMODES 61
typedef struct sph_stir_params {
  double sigma;             /* stationary rms of each OU component                 */
  double t_decay;           /* OU correlation time                                 */
  double sol_weight;        /* zeta: 1 = solenoidal, 0 = compressive               */
} sph_stir_params;

typedef struct sph_ctx sph_ctx;

/* --- configuration and lifetime --------------------------------------------- */

/* Fills *cfg with the defaults of SURVEY 8(c): unit periodic box [-0.5,0.5]^3,
 * ideal gas gamma 5/3, exact K, ng0 100, ngmax 150, L <= 8, h_cap 0.25, C 0.2,
 * growth 1.1, dt_first 1e-6, alpha 1, beta 2, eps 0.01.  Pure. */
int sph_config_default(sph_config* cfg);

/* Bytes of device arena needed for cfg (pure; no CUDA call). */
int sph_workspace_size(const sph_config* cfg, size_t* bytes);

/* Creates a context on cfg->device using the caller's arena (device pointer,
 * >= sph_workspace_size bytes, 256-B aligned) and stream (cudaStream_t, may be
 * NULL for the legacy stream).  Initialises NVML when available. */
int sph_init(const sph_config* cfg, void* arena, size_t arena_bytes, void* stream, sph_ctx** out);

/* Resets any locked clock this context set (NVML), releases host bookkeeping.
 * The arena is the caller's to free afterwards.  NULL is a no-op. */
void sph_finalize(sph_ctx* ctx);

const char* sph_last_error(const sph_ctx* ctx);
const char* sph_phase_name(int phase);

/* --- particle I/O ------------------------------------------------------------ */

/* Copies n particles in (mem = SPH_MEM_HOST or SPH_MEM_DEVICE pointers, each an
 * array of n values).  du_m1 may be NULL (zeros); id may be NULL (0..n-1).
 * n > n_capacity -> SPH_ERR_CAPACITY.  n = 0 is allowed (every phase is then a
 * no-op and sph_step returns dt = growth * dt_prev).  Resets the stage machine
 * to "particles set".  Periodic coordinates must lie in [box_min, box_max]. */
int sph_set_particles(sph_ctx* ctx, int64_t n, const double* x, const double* y, const double* z,
                      const double* vx, const double* vy, const double* vz, const double* h,
                      const double* m, const double* u, const double* du_m1, const int64_t* id,
                      int mem);

/* Sets the integrator clock: current time, dt of the previous step (dt_m1 of
 * item 10) and whether the next step is the first (du_m1 := du). */
int sph_set_time(sph_ctx* ctx, double t, double dt_prev, int first_step);
int sph_get_time(sph_ctx* ctx, double* t, double* dt_prev, int* first_step);

int sph_get_n(const sph_ctx* ctx, int64_t* n);

/* Copies field f (n values; int64 for SPH_F_ID, uint64 for SPH_F_KEY, int32 for
 * SPH_F_NC, double otherwise) to dst (host or device).  Synchronises, except
 * with SPH_MEM_HOST_ASYNC (valid after sph_sync). */
int sph_get_field(sph_ctx* ctx, int field, void* dst, int mem);

/* Waits for everything enqueued on the context's stream. */
int sph_sync(sph_ctx* ctx);

/* Multi-GPU halo support (SFC domain decomposition).  A particle
 * whose id has bit SPH_GHOST_BIT set is a ghost: a copy of a particle owned by
 * another rank, present only as a neighbour j.  Its own sums use an incomplete
 * neighbourhood and are meaningless (the IAD singularity check ignores ghosts);
 * the owners' values are written over it with sph_set_field:
 *   after sph_density:  SPH_F_RHO           (then sph_eos derives p, c, V);
 *   after sph_iad:      SPH_F_C11..SPH_F_C33 and, with cfg.av_switch, SPH_F_BAL
 *                       (the momentum records are rebuilt).
 * sph_set_field copies n values (current order) from src; only SPH_F_RHO,
 * SPH_F_C11..SPH_F_C33 and SPH_F_BAL are settable (SPH_ERR_ARG otherwise). */
#define SPH_GHOST_BIT (1ll << 62)
int sph_set_field(sph_ctx* ctx, int field, const void* src, int mem);

/* The local min_i h_i/c_i of the last sph_momentum_energy (synchronises), and
 * the global one (the minimum over ranks, the P:220 collective) to be used by
 * the next sph_timestep instead. */
int sph_get_local_min_hc(sph_ctx* ctx, double* min_hc);
int sph_set_global_min_hc(sph_ctx* ctx, double min_hc);

/* Device-side plumbing of the decomposed step ("domain
 * decomposition, halo exchanges", P:216 DomainDecompAndSync).  They move and
 * select particles; none changes a value of the method.  All pointers are
 * DEVICE pointers on cfg.device except `boxes`; indices refer to the current
 * particle order.  A row is SPH_ROW_DOUBLES doubles
 * {x, y, z, vx, vy, vz, h, m, u, du_m1, id (int64 bit pattern)}.
 *
 * sph_compute_keys: phase KEYS alone (box + Morton keys) in the CURRENT order,
 *   no sort; SPH_F_KEY then returns them (the SFC partition reads them).
 * sph_compact: stable in-place compaction keeping particle i iff
 *   (keep == NULL || keep[i] != 0) && !(drop_ghosts && (id[i] & SPH_GHOST_BIT));
 *   *n_out = new count.  Synchronises.
 * sph_pack_rows: rows of particles idx[0..m) into dst [m][SPH_ROW_DOUBLES],
 *   id OR-ed with or_id (SPH_GHOST_BIT marks ghosts).
 * sph_append_rows: m rows after the current n particles (n + m <= n_capacity,
 *   else SPH_ERR_CAPACITY).
 * sph_select_ghosts: mask[i] bit r (r < R <= 64, r != self) set iff particle i
 *   is closer than `radius` (minimum image on periodic axes) to the box
 *   boxes[6r..6r+5] = {lo_x, lo_y, lo_z, hi_x, hi_y, hi_z} (host array) of rank r;
 *   an empty box (lo > hi) selects nothing.
 * sph_gather_field / sph_scatter_field: dst[k] = f[idx[k]] / f[idx[k]] = src[k]
 *   for a double field; scatter follows sph_set_field's rules (settable fields
 *   and stages) and also accepts SPH_F_OMEGA after sph_gradh.
 * SPH_F_ORDER (int32, via sph_get_field): after sph_build_tree, the pre-sort
 *   index of the particle now at each position (the sort's permutation).
 * compact / append leave the context at the "particles set" stage. */
#define SPH_ROW_DOUBLES 11
int sph_compute_keys(sph_ctx* ctx);
int sph_compact(sph_ctx* ctx, const uint8_t* keep, int drop_ghosts, int64_t* n_out);
int sph_pack_rows(sph_ctx* ctx, const int64_t* idx, int64_t m, uint64_t or_id, double* dst);
int sph_append_rows(sph_ctx* ctx, const double* rows, int64_t m);
int sph_select_ghosts(sph_ctx* ctx, const double* boxes, int R, int self, double radius,
                      uint64_t* mask);
int sph_gather_field(sph_ctx* ctx, int field, const int64_t* idx, int64_t m, double* dst);
int sph_scatter_field(sph_ctx* ctx, int field, const int64_t* idx, int64_t m, const double* src);

/* --- SFC decomposition on the device ----------
 * decomp.py issues the collectives (all-reduce, all-to-all over NCCL) between
 * these calls; every selection, count, split, pack and map runs here.  All
 * pointers are DEVICE pointers owned by the caller; all calls are asynchronous
 * on the context's stream.  Ranks <= 64.
 *
 * sph_decomp_reduce: red[0..6] = (-min x, -min y, -min z, max x, max y, max z,
 *   max h) over the held particles that are not ghosts (-inf when none).  An
 *   element-wise MAX all-reduce of red over the ranks gives the global bounding
 *   box and h_max exactly.
 * sph_set_key_box: from now on the KEYS phase uses [-red[a], red[3 + a]] as the
 *   box of every OPEN axis a (periodic axes keep the configured box) and red[6]
 *   as h_max for sph_decomp_ghosts -- the all-reduced red makes every rank's
 *   keys those of the single-GPU run.  red == NULL: each step's own box again.
 * sph_key_histogram: hist[b] (int64, 2^bits) = held non-ghost particles whose
 *   key has top bits b (after sph_compute_keys; bits a multiple of 3).
 * sph_decomp_owners: (ghosts held from the last step are skipped: mask 0,
 *   not counted) from the histogram summed over ranks, the split bins
 *   s_0 = 0 <= s_1 <= .. <= s_world = 2^bits with s_r = the first bin whose
 *   inclusive prefix count exceeds floor(total r / world); rank r owns the keys
 *   of bins [s_r, s_r+1).  mig_mask[i] = 1 << owner(i) if owner(i) != rank
 *   else 0; counts[r] (int64, world) = held particles owned by r.  The splits
 *   are kept for sph_decomp_ghosts.
 * sph_decomp_ghosts: L = the finest level whose cells have side >= 2 h_max
 *   (sph_set_key_box) on every axis; mask[i] = the ranks (except `rank`) owning
 *   a key of one of the 27 level-L cells around particle i's (periodic wrap,
 *   clipped at open faces); counts[r] = particles with bit r.  Every particle
 *   within 2 h_max of a particle owned by r has bit r: the halo is conservative.
 * sph_decomp_pack: one row per (particle i, rank r in mask[i]), grouped by r in
 *   rank order and in particle order within r (id OR-ed with or_id);
 *   pos[e] = i of row e.  rows/pos hold sum_i popcount(mask[i]) entries.
 * sph_decomp_drop: stable compaction keeping the non-ghosts with
 *   drop_mask[i] == 0 (drop_mask may be NULL; n_expected == n: nothing to
 *   do); the new count is the caller's n_expected (from the
 *   counts, no synchronisation); a different device count is reported as
 *   SPH_ERR_STATE at the next synchronising call.
 * sph_decomp_map: after sph_build_tree, the positions after its sort of the
 *   positions pre[k] before it (pre == NULL: first + k), for the halo lists.
 * sph_halo_gather / sph_halo_scatter: rows [m][nf] of the fields at idx; the
 *   scatter takes the same fields and refreshes what depends on them, as
 *   sph_scatter_field does.
 * sph_min_hc_dev / sph_set_min_hc_dev: the local min h/c (or h/v_sig) of the
 *   last MOMENTUM_ENERGY into / the global minimum from a device double (the
 *   P:220 collective without a host round trip). */
int sph_decomp_reduce(sph_ctx* ctx, double* red);
int sph_set_key_box(sph_ctx* ctx, const double* red);
int sph_key_histogram(sph_ctx* ctx, int bits, int64_t* hist);
int sph_decomp_owners(sph_ctx* ctx, const int64_t* hist, int bits, int rank, int world, uint64_t* mig_mask,
                      int64_t* counts);
int sph_decomp_ghosts(sph_ctx* ctx, int bits, int rank, int world, uint64_t* mask, int64_t* counts);
int sph_decomp_pack(sph_ctx* ctx, const uint64_t* mask, int world, uint64_t or_id, double* rows, int64_t* pos);
int sph_decomp_drop(sph_ctx* ctx, const uint64_t* drop_mask, int64_t n_expected);
int sph_decomp_map(sph_ctx* ctx, const int64_t* pre, int64_t first, int64_t m, int64_t* post);
int sph_halo_gather(sph_ctx* ctx, const int32_t* fields, int nf, const int64_t* idx, int64_t m, double* dst);
int sph_halo_scatter(sph_ctx* ctx, const int32_t* fields, int nf, const int64_t* idx, int64_t m,
                     const double* src);
int sph_min_hc_dev(sph_ctx* ctx, double* dst);
int sph_set_min_hc_dev(sph_ctx* ctx, const double* src);

/* Split IAD / MOMENTUM_ENERGY for overlapping the halo exchanges with compute
 * (SURVEY 8(e)): the neighbour search flags every target that has a ghost among
 * its neighbours.  With part INTERIOR, sph_iad / sph_momentum_energy process
 * only the targets without one (they need no halo value) and leave the stage
 * unchanged; BOUNDARY processes the rest (and the ghosts' momentum records in
 * IAD) and advances the stage; ALL (default) is the plain call.  GHOSTS makes
 * sph_eos recompute only the ghosts (after their rho arrived).  Each target is
 * computed once with the same inputs, so the results equal the unsplit step
 * bit for bit.  Not with grad-h / volume elements (SPH_ERR_NOT_SUPPORTED). */
enum { SPH_PART_ALL = 0, SPH_PART_INTERIOR = 1, SPH_PART_BOUNDARY = 2, SPH_PART_GHOSTS = 3 };
int sph_set_part(sph_ctx* ctx, int part);

/* --- the hot path (each call = one accounted phase group) ------------------- */

/* Items 1-3: box (open axes: exact min/max), 63-bit Morton keys, stable LSD
 * radix sort (onesweep, 8 x 8-bit digits) and permutation of every particle
 * field into key order; then the cell table (level L = finest with cell side >=
 * 2 h_max on every axis, L <= max_cell_level).  Phases KEYS, SORT, CELLS. */
int sph_build_tree(sph_ctx* ctx);

/* Item 4: j in N(i) iff j != i and d2 < (2 h_i)^2 with d the minimum image,
 * d2 = (dx*dx + dy*dy) + dz*dz rounded per operation (bit-exact vs brute force).
 * Lists are ascending in the current order.  Fills *stats when non-NULL
 * (synchronises).  max nc > ngmax -> SPH_ERR_CAPACITY, stats.max_nc = needed. */
int sph_find_neighbors(sph_ctx* ctx, sph_nbr_stats* stats);

/* Copies the neighbour lists to host CSR: offsets[n+1] (int64), idx (int32,
 * current-order indices, ascending per particle).  idx_cap < total ->
 * SPH_ERR_CAPACITY with offsets still filled. */
int sph_get_neighbors(sph_ctx* ctx, int64_t* offsets, int32_t* idx, int64_t idx_cap);

/* The lists of nt chosen particles only (current-order indices `targets`):
 * offsets[nt+1], idx as in sph_get_neighbors.  For sampled checks at full size. */
int sph_get_neighbor_rows(sph_ctx* ctx, const int64_t* targets, int64_t nt, int64_t* offsets,
                          int32_t* idx, int64_t idx_cap);

/* Item 5 (XMass): rho_i = (K/h_i^3) [m_i + sum_j m_j S(pi r_ij/2h_i)^6].  DENSITY. */
int sph_density(sph_ctx* ctx);

/* Item 6: ideal p = (gamma-1) rho u, c = sqrt(gamma (gamma-1) u); isothermal
 * p = c0^2 rho, c = c0.  EOS. */
int sph_eos(sph_ctx* ctx);

/* Item 7 (IADVelocityDivCurl): tau_i = sum_j (m_j/rho_j) W(r,h_i)
 * Delta Delta^T, C_i = tau_i^{-1} (adjugate).  With cfg.divcurl the same pass
 * accumulates M_i = sum_j V_j W Delta (v_j - v_i)^T and forms the IAD velocity
 * gradient T_i = C_i M_i (T_ab = dv_b/dx_a; exact for linear fields): div v =
 * tr T, curl v = (T_yz - T_zy, T_zx - T_xz, T_xy - T_yx); with cfg.av_switch
 * also the Balsara factor f_i = |div| / (|div| + |curl| + 1e-4 c_i/h_i) that
 * scales the AV of a pair by (f_i + f_j)/2 in MOMENTUM_ENERGY (reading 19).
 * SPH_ERR_SINGULAR is reported at the next synchronising call.  IAD. */
int sph_iad(sph_ctx* ctx);

/* Item 8 (MomentumEnergy): a_i, du_i with IAD gradients and Monaghan AV, plus
 * the local min_i h_i/c_i for item 9.  MOMENTUM_ENERGY. */
int sph_momentum_energy(sph_ctx* ctx);

/* Item 9: dt = min(C min_i h_i/c_i, growth dt_prev).  Synchronises; *dt may be
 * NULL.  TIMESTEP. */
int sph_timestep(sph_ctx* ctx, double* dt);

/* Item 10: kick, drift (+ periodic wrap), AB2 energy update, h update; advances
 * t and dt_prev.  UPDATE. */
int sph_update(sph_ctx* ctx);

/* Items 1-10 in order; legal whenever particles are set.  Synchronises once at
 * the end (plus at every phase edge with PHASE accounting). */
int sph_step(sph_ctx* ctx, sph_step_info* info);

/* --- energy and clocks ------------------------------------------- */

/* Clock policy: DEFAULT, STATIC (mhz[0] for every phase) or PER_PHASE (mhz[p]
 * set before phase p, skipped when unchanged; 0 = leave the clock as is).
 * NVML applies a lock when it is called, not in stream order, so PER_PHASE
 * synchronises the stream before every clock change (each phase then runs at
 * its own clock; the wait is part of the policy's time, as the paper's
 * ManDyn includes its clock-switch latency).
 * Requests snap to the nearest supported graphics clock.  Uses
 * nvmlDeviceSetGpuLockedClocks; this needs root and is disabled unless the
 * environment sets SPH_ALLOW_CLOCK_CONTROL=1 (shared hosts forbid clock changes)
 * -> SPH_ERR_NO_PERMISSION / SPH_ERR_NOT_SUPPORTED leave the policy DEFAULT. */
int sph_set_clock_policy(sph_ctx* ctx, int mode, const uint32_t mhz[SPH_NPHASES]);

/* The SM (graphics) clocks the device supports at its highest memory clock,
 * descending (NVML nvmlDeviceGetSupportedGraphicsClocks) -- the candidate set of
 * the per-function frequency search (Fig. 2).  *n = count (<= cap).
 * SPH_ERR_NVML when NVML is unavailable.  Does not change any clock. */
int sph_supported_clocks(sph_ctx* ctx, uint32_t* mhz, int cap, int* n);

/* One row per phase (cap >= SPH_NPHASES).  Time is always filled; joules only
 * with PHASE accounting and a working NVML energy counter. */
int sph_energy_report(sph_ctx* ctx, sph_energy_row* rows, int cap, int* n_rows);
/* Zeroes the rows and the PHASE accumulators and reads the energy counter as
 * the start of the accounting window. */
int sph_energy_reset(sph_ctx* ctx);

/* The accounting window since sph_energy_reset (synchronises): the sampled
 * energy (sum over phases + between phases), the NVML total-energy counter
 * delta over the same window (-1 when unreadable; the counter advances in
 * ~100 ms / ~99 J steps on a B200, so windows of >= 10 s keep it within 1%),
 * wall and sampled seconds.  sampled_joules vs counter_joules is the
 * accounting's self-check (SURVEY 8(c) "Energy accounting"). */
typedef struct sph_energy_window {
  double wall_seconds;
  double sampled_seconds;
  double sampled_joules;
  double between_joules;    /* sampled while no phase was running (host gaps)  */
  double counter_joules;
  int64_t samples;
} sph_energy_window;
int sph_energy_totals(sph_ctx* ctx, sph_energy_window* totals);

/* Total-energy counter of the device in mJ (NVML), for whole-run deltas. */
int sph_energy_counter_mj(sph_ctx* ctx, uint64_t* mj);

/* Switches the accounting mode of an existing context (sph_accounting_mode). */
int sph_set_accounting(sph_ctx* ctx, int mode);

/* Number of libsph kernels launched by this process so far (all contexts);
 * for the bench's launch count. */
int sph_kernel_launches(int64_t* count);

/* Re-runs one phase reps times back to back on the same inputs -- the
 * KernelTuner-style isolated measurement of P:81-87 -- and returns its mean time
 * and energy per call (joules < 0 when NVML is unavailable).  Repeatable phases
 * leave the pipeline state unchanged: KEYS (into a spare key buffer), SORT
 * (re-sorts the sorted keys, permutes into the spare state buffer; the last
 * permutation, SPH_F_ORDER, is saved and restored), CELLS, NEIGHBORS, DENSITY,
 * EOS (after GRADH with p/(Omega rho^2), as the pipeline left it), IAD,
 * MOMENTUM_ENERGY, TIMESTEP, GRADH (cfg.gradh without cfg.ve); UPDATE is not
 * (SPH_ERR_ARG).  DENSITY after the volume-element GRADH would overwrite the
 * normalised rho: SPH_ERR_STATE.  The NVML energy counter of a B200 advances about every 100 ms,
 * so reps should make the call last >= 1 s.  Synchronises. */
int sph_repeat_phase(sph_ctx* ctx, int phase, int reps, double* ms_per_call,
                     double* joules_per_call);

/* --- NormalizationGradh and the signal-velocity time step -- */

/* Phase GRADH (NormalizationGradh; reading 21 of DESIGN.md, the paper
 * prints no formula): Omega_i = 1 + (h_i / (3 rho_i)) sum_j m_j dW(r_ij, h_i)/dh_i
 * over the neighbour list plus the self term (dW/dh = -(K/h^4) S^5 (6 cos x - 3 S),
 * x = pi r / 2h), i.e. 1 + (h/3rho) d rho/dh.  Writes Omega (SPH_F_OMEGA) and
 * replaces p/rho^2 by p/(Omega rho^2) in the momentum-energy terms.  Needs
 * cfg.gradh; after sph_eos, before sph_iad (sph_iad returns SPH_ERR_STATE while
 * it is pending).  sph_step runs it when cfg.gradh.  With cfg.dt_vsig the
 * momentum-energy phase also forms vsig_i = max(2 c_i, max_j (c_i + c_j - 3 w_ij)),
 * w_ij = min(0, v_ij . d_ij / r_ij) (SPH_F_VSIG), and the time step becomes
 * dt = min(C min_i h_i / vsig_i, growth dt_prev) (reading 22).
 * With cfg.ve (generalized volume elements, reading 23) the same phase first
 * forms X_i = m_i / rho0_i (rho0 = the density of sph_density), the
 * normalisation kx_i = (K/h_i^3)[X_i + sum_j X_j S^6] and rho_i = kx_i m_i / X_i,
 * Omega with X and kx in place of m and rho, and re-runs the EOS on the new
 * density (p / (Omega rho^2) when cfg.gradh).  sph_step runs it when cfg.gradh
 * or cfg.ve. */
int sph_gradh(sph_ctx* ctx);

/* --- self-gravity ------------------------------------------ */

/* Phase GRAVITY (the Evrard collapse's extra function; reading
 * 20): a_i += G sum_j m_j (x_j - x_i) / (|x_j - x_i|^2 + eps^2)^(3/2) and the
 * potential phi_i, by a Barnes-Hut walk of the Morton octree (levels 0..Lt,
 * monopole + traceless quadrupole per cell, a cell is used as a multipole when
 * its side < theta * distance from the 32 targets' box to its centre of mass;
 * leaves not accepted are summed directly).  theta = 0 is exact direct
 * summation in ascending particle order.  Needs cfg.gravity (arena room for the
 * octree) and a fully open box; after sph_momentum_energy.  Runs inside sph_step
 * when enabled. */
int sph_gravity(sph_ctx* ctx);

/* --- turbulence driving ------------------------------------ */

/* The fixed mode set: writes 3 * SPH_STIR_NMODES ints (n_x, n_y, n_z per mode)
 * to n3 (cap >= SPH_STIR_NMODES modes) and returns the mode count.  Pure. */
int sph_stir_modes(int32_t* n3, int cap);

/* Enables driving: per-mode weights w[SPH_STIR_NMODES], the initial OU state
 * A0[6 * SPH_STIR_NMODES] (NULL = zeros) and the noise table
 * noise[nsteps][SPH_STIR_NMODES][6] (nsteps <= cfg.stir_steps; host or device
 * pointers per mem).  Resets the step counter.  cfg.stir_steps == 0 ->
 * SPH_ERR_NOT_SUPPORTED.  Once enabled, sph_step runs STIR after
 * MOMENTUM_ENERGY; a step past the end of the noise table -> SPH_ERR_CAPACITY
 * at the next synchronising call. */
int sph_stir_init(sph_ctx* ctx, const sph_stir_params* prm, const double* w, const double* A0,
                  const double* noise, int64_t nsteps, int mem);

/* Phase STIR alone (after sph_momentum_energy, before sph_timestep): the OU
 * update with the previous step's dt and the driving acceleration added to
 * a_i.  SPH_ERR_STATE when driving is not enabled. */
int sph_stir(sph_ctx* ctx);

/* The OU state A (6 * SPH_STIR_NMODES doubles, host) and the number of STIR
 * phases run since sph_stir_init.  Synchronises. */
int sph_stir_get_state(sph_ctx* ctx, double* A, int64_t* steps);

/* DVFS trace (Fig. 9).  sph_trace_start launches a host thread that
 * samples NVML (SM clock, power, energy counter) every period_ms (>= 0.1; a
 * sample is taken back to back when the NVML queries themselves take longer --
 * several ms on a B200 host, see query_us) into a
 * buffer of `capacity` samples, each tagged with the phase the device is running:
 * while a trace is active, every phase writes its id (and -1 when it ends) into
 * a pinned, device-mapped host word from the stream (one 1-thread kernel per
 * edge, so the tag follows the device, not the asynchronous host).  The pinned
 * word (4 bytes, cudaHostAlloc) is the only allocation the library makes.
 * SPH_ERR_NVML when NVML is unavailable, SPH_ERR_STATE if a trace is running.
 * sph_trace_stop joins the thread and copies min(cap, taken) samples in time
 * order to `out` (may be NULL with cap = 0 to discard); *n = samples taken. */
int sph_trace_start(sph_ctx* ctx, double period_ms, int64_t capacity);
int sph_trace_stop(sph_ctx* ctx, sph_trace_sample* out, int64_t cap, int64_t* n);

#ifdef __cplusplus
}
#endif
#endif /* SPH_H */
