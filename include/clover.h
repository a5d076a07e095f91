/*
 * clover.h -- C ABI of the B200-native CloverLeaf 2D timestep library
 * (libclover.so, built from paper_conf_cluster_regulymg15_b200/csrc/).
 *
 * What the library computes: the hot path named by BASELINE.json north_star,
 * i.e. one CloverLeaf 2D explicit Lagrangian-remap timestep of the
 * compressible Euler equations on a structured staggered fp64 mesh ("a
 * system of four partial differential equations ... conservation of energy,
 * density and momentum ... finite volume method on a structured staggered
 * grid", sec. V), with the step arithmetic read as in
 * SURVEY.md sec. 8(c) c.1-c.13.  The interface
 * follows the paper's problem statement: the mesh and its data are declared
 * once and "all data is handed over to the library" behind an opaque handle
 * (sec. II.A, sec. II.C).
 *
 * Conventions
 *  - Every function returns an int status: CLOVER_OK (0) or a negative
 *    CLOVER_ERR_* code.  No C++ exception crosses this boundary.
 *  - Indices: j = x index, k = y index, 1-based interior, logical halo 2.
 *  - Host field arrays use the GLOBAL INTERIOR, row-major, j fastest:
 *      cells nx*ny, nodes (nx+1)*(ny+1), x-faces (nx+1)*ny, y-faces nx*(ny+1).
 *  - Device memory: the caller hands the library ONE device workspace
 *    (e.g. a torch.uint8 tensor) of at least clover_workspace_bytes(); the
 *    library carves all fields from it and never allocates device memory
 *    itself.  The caller owns the workspace and must keep it alive until
 *    clover_finalize().  Structs and host buffers passed in are copied; the
 *    caller keeps ownership.
 *  - Streams: all device work is enqueued on the cudaStream_t passed to
 *    clover_init (NULL = legacy default stream).  clover_step is
 *    asynchronous; errors detected on the device (small dt, negative
 *    volume in PdV) are latched (the first one wins) and
 *    returned by the next synchronising call (clover_field_summary,
 *    clover_get_clock, clover_read_field, clover_sync, clover_finalize).
 *  - Multi-GPU: one process per GPU; the mesh is 2D-block decomposed into
 *    px*py chunks ("partitioning across processes and ...
 *    standard halo exchanges"); ranks exchange depth-2 halos with NCCL
 *    send/recv and reduce dt with an NCCL MIN all-reduce.  A single process
 *    may also own several chunks ("local chunks"), exchanged with
 *    device-to-device copies; results are bitwise identical for every
 *    decomposition.
 */
#ifndef CLOVER_H
#define CLOVER_H
#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define CLOVER_ABI_VERSION 2  /* 2: clover_dist.host_transport */

enum {
  CLOVER_OK = 0,
  CLOVER_ERR_ARG = -1,        /* invalid argument (message: clover_last_error) */
  CLOVER_ERR_CUDA = -2,       /* a CUDA runtime call failed */
  CLOVER_ERR_NCCL = -3,       /* an NCCL call failed or NCCL is unavailable */
  CLOVER_ERR_WORKSPACE = -4,  /* workspace too small or misaligned */
  CLOVER_ERR_SMALL_DT = -5,   /* dt < dtmin: the reference's "small timestep" abort */
  CLOVER_ERR_NEG_VOLUME = -6, /* PdV corrector: volume + total_flux is not
                                 > 0 in some cell (negative volume, or NaN in the fluxes);
                                 latched on the device, the step's results are invalid */
  CLOVER_ERR_STATE = -7,      /* call not valid in the current state */
  CLOVER_ERR_NAN = -8         /* clover_field_summary: a total is NaN */
};

enum { CLOVER_GEOM_RECT = 1, CLOVER_GEOM_CIRCLE = 2, CLOVER_GEOM_POINT = 3 };

/* Tangential mirror of face fields at walls (reading A7). */
enum { CLOVER_MIRROR_GEOMETRIC = 0, CLOVER_MIRROR_CELLCENTRE = 1 };

/* Mesh and run parameters (SURVEY 2d D6 input deck).  A zero in any of
 * dtinit/dtmax/dtmin/dtrise/dt*_safe selects the CloverLeaf default
 * 0.1 / 1.0 / 1e-7 / 1.5 / (0.7, 0.5, 0.5, 0.7). */
typedef struct {
  int32_t x_cells, y_cells;         /* global mesh, >= 4 each */
  double xmin, ymin, xmax, ymax;    /* domain, xmax > xmin, ymax > ymin */
  double dtinit, dtmax, dtmin, dtrise;
  double dtc_safe, dtu_safe, dtv_safe, dtdiv_safe;
  int32_t advect_x_first;           /* 1: x sweep first on step 1 (reference) */
  int32_t face_mirror;              /* CLOVER_MIRROR_* */
} clover_grid;

/* One entry of the state list.  states[0] is the background and fills the
 * whole mesh; later states are painted in order.
 * Rectangle: [xmin,xmax]x[ymin,ymax]; circle: centre (xmin,ymin) + radius;
 * point: the vertex (xmin,ymin). */
typedef struct {
  double density, energy, xvel, yvel;
  int32_t geometry;                 /* CLOVER_GEOM_* (ignored for states[0]) */
  double xmin, xmax, ymin, ymax, radius;
} clover_state;

/* Host transport (S:8(e), "standard halo exchanges"): the three
 * collectives of a multi-rank step carried by caller callbacks on HOST
 * buffers instead of NCCL -- for several ranks without NCCL (e.g. processes
 * sharing one GPU, which NCCL refuses).  Every callback returns 0 on
 * success; the library copies device data to host before a call and back
 * after it, synchronously (CUDA graphs are off in this mode).
 *  sendrecv: for i in [0, n): send send[i] (nsend[i] doubles) to rank
 *    peer[i] and receive recv[i] (nrecv[i] doubles) from rank peer[i];
 *    several messages to one peer are matched in list order.
 *  allreduce_min_u64: *value = min over ranks (dt bit pattern, in place).
 *  allgather_f64: recv[r*count .. ] = rank r's send (count doubles each). */
typedef struct {
  void* user;
  int (*sendrecv)(void* user, int32_t n, const int32_t* peer, const double* const* send,
                  const int64_t* nsend, double* const* recv, const int64_t* nrecv);
  int (*allreduce_min_u64)(void* user, uint64_t* value);
  int (*allgather_f64)(void* user, const double* send, int64_t count, double* recv);
} clover_host_transport;

/* Decomposition.  nranks processes, each owning chunks_x*chunks_y/nranks
 * chunks of a px*py chunk grid (px = chunks in x).  nranks==1 with
 * px*py>1 runs all chunks on one GPU.  nccl_unique_id: 128 bytes from
 * clover_nccl_unique_id() on rank 0, broadcast by the caller; NULL when
 * nranks == 1 or when host_transport is given (then NCCL is not used;
 * the struct is copied, its callbacks must outlive the context). */
typedef struct {
  int32_t rank, nranks;
  int32_t px, py;
  const void* nccl_unique_id;
  const clover_host_transport* host_transport; /* NULL = NCCL */
} clover_dist;

/* field_summary totals: density = mass/vol,
 * pressure = press/vol, total energy = ie + ke. */
typedef struct {
  double vol, mass, ie, ke, press;
} clover_summary;

/* Field ids for clover_read_field / clover_write_field. */
enum {
  CLOVER_F_DENSITY0 = 0,  /* cell  */
  CLOVER_F_ENERGY0 = 1,   /* cell  */
  CLOVER_F_PRESSURE = 2,  /* cell, = ideal_gas(density0, energy0) at read time */
  CLOVER_F_VISCOSITY = 3, /* cell, artificial viscosity of the last step */
  CLOVER_F_SOUNDSPEED = 4,/* cell, = ideal_gas(density0, energy0) at read time */
  CLOVER_F_XVEL0 = 5,     /* node */
  CLOVER_F_YVEL0 = 6,     /* node */
  CLOVER_F_VOL_FLUX_X = 11,  /* x-face, volume flux of the last step */
  CLOVER_F_VOL_FLUX_Y = 12,  /* y-face */
  CLOVER_F_MASS_FLUX_X = 13, /* x-face, mass flux of the last x sweep */
  CLOVER_F_MASS_FLUX_Y = 14  /* y-face, mass flux of the last y sweep */
};

typedef struct clover_ctx clover_ctx;

/* Bytes of device workspace clover_init needs for this grid/decomposition
 * on this rank (all local chunks).  dist may be NULL (1 chunk). */
int clover_workspace_bytes(const clover_grid* grid, const clover_dist* dist, int64_t* bytes);

/* 128-byte NCCL unique id for a multi-process run (call on rank 0 only). */
int clover_nccl_unique_id(void* out128);

/* Create a context: carve fields from `workspace`, paint the states
 * (generate_chunk), compute the EOS and prime all halos (start of run,
 * SURVEY 8(c) c.1).  Validation: x_cells,y_cells >= 4; nstates >= 1;
 * xmax > xmin; ymax > ymin; px*py >= nranks and divisible by nranks; every
 * chunk at least 4x4 cells.  On error *out is NULL.
 * Multi-rank NCCL contexts with CLOVER_LSA=1 in every rank's environment
 * exchange halos by device-initiated stores into the peers' NCCL symmetric
 * windows (see clover_debug_set_virtual_remote, enable = 3); the library
 * then allocates its mailbox with ncclMemAlloc (collective, freed by
 * clover_finalize); CLOVER_ERR_NCCL if not every rank is load/store
 * reachable. */
int clover_init(const clover_grid* grid, const clover_state* states, int32_t nstates,
                const clover_dist* dist, void* workspace, int64_t workspace_bytes,
                void* cuda_stream, clover_ctx** out);

/* Advance nsteps full timesteps (SURVEY 3(ii) hydro loop: timestep, PdV
 * predictor, accelerate, PdV corrector, flux_calc, advection sweeps,
 * reset_field).  Asynchronous on the context stream; no host sync. */
int clover_step(clover_ctx* ctx, int32_t nsteps);

/* End-to-end entry with HOST buffers: copy the state density0, energy0
 * (cells), xvel0, yvel0 (nodes) from host memory (pinned for speed) into the
 * mesh, advance nsteps, copy the four state fields back to host_out (may
 * alias host_in).  Synchronous.  The host arrays are the global interiors
 * (row-major, j fastest); with several chunks each process moves the owned
 * blocks of its own chunks (a multi-rank call is collective, and a rank's
 * arrays outside its chunks are neither read nor written).  A NULL input
 * keeps that field's current values; a NULL output is not copied back. */
int clover_step_host(clover_ctx* ctx, int32_t nsteps,
                     const double* density0_in, const double* energy0_in,
                     const double* xvel0_in, const double* yvel0_in,
                     double* density0_out, double* energy0_out,
                     double* xvel0_out, double* yvel0_out);

/* Global field_summary over all chunks and ranks; synchronises.  The
 * reduction is deterministic: each 16x16-cell tile aligned to the global
 * index is reduced in a fixed order on the device (row sums by warp
 * shuffles, then a fixed tree), and the tile partials are summed in global
 * tile order on the host, so every decomposition gives the same bits.
 * Returns CLOVER_ERR_NAN (the totals are still written) if a total is NaN,
 * else a latched device error if any.  Multi-rank contexts all-gather the
 * tile partials through a temporary device buffer (an I/O path, like
 * clover_read_field). */
int clover_field_summary(clover_ctx* ctx, clover_summary* out);

/* Step counter, simulated time and the last dt; synchronises. */
int clover_get_clock(clover_ctx* ctx, int32_t* step, double* time, double* dt_last);

/* dt of steps [first, first+n) (1-based step numbers, last 4096 kept).
 * After clover_restart only steps after the checkpoint's step are known:
 * earlier ones are rejected with CLOVER_ERR_ARG. */
int clover_dt_history(clover_ctx* ctx, int32_t first, int32_t n, double* host_out);

/* Gather a field's global interior into host memory (n = element count of
 * the field's kind, see above).  Every rank receives the full field
 * (multi-rank: NCCL all-gather through a temporary device buffer -- the one
 * place the library allocates device memory, a debug/I-O path). */
int clover_read_field(clover_ctx* ctx, int32_t field_id, double* host, int64_t n);

/* Read a w x h window of a field's global interior, starting at global
 * 1-based index (j0, k0), into host (row-major, j fastest, w*h doubles);
 * PRESSURE / SOUNDSPEED are evaluated from the current state as above.  The
 * window must lie inside the field's interior (nx*ny cells, (nx+1)*(ny+1)
 * nodes, ...), else CLOVER_ERR_ARG.  Single-process contexts (any number of
 * local chunks); CLOVER_ERR_STATE for nranks > 1.  Synchronises.  For
 * inspecting part of a mesh too large to copy whole to the host. */
int clover_read_field_window(clover_ctx* ctx, int32_t field_id, int32_t j0, int32_t k0, int32_t w,
                             int32_t h, double* host);

/* Overwrite the global interior of a state field (DENSITY0, ENERGY0, XVEL0,
 * YVEL0) from host memory and refresh its halos. */
int clover_write_field(clover_ctx* ctx, int32_t field_id, const double* host, int64_t n);

/* Wait for all queued work; returns a latched device error if any. */
int clover_sync(clover_ctx* ctx);

/* Use CUDA graphs for clover_step (default on).  0 = direct launches. */
int clover_set_graphs(clover_ctx* ctx, int32_t enable);

/* Number of CUDA kernels one clover_step(ctx, 1) launches on this rank. */
int clover_kernels_per_step(clover_ctx* ctx, int32_t* out);

/* Step kernels (streaming kernels, IEEE fixups, wall bands; not the halo
 * strip copies) launched on this context so far by clover_step,
 * clover_profile_steps and clover_debug_partial_step; a graph launch counts
 * the kernels captured in it.  The bench's gpu_launches is the difference
 * across its timed region. */
int clover_launch_count(clover_ctx* ctx, int64_t* out);

/* Bounding box of this process's chunks in global cell indices: out4 =
 * {j0, k0, width, height} (0-based origin; cells [j0, j0+width) x
 * [k0, k0+height)).  E.g. to pin only the rows of the global host arrays
 * that clover_step_host moves on this rank. */
int clover_local_block(clover_ctx* ctx, int32_t* out4);

/* Profiling: run nsteps full steps with direct launches and a CUDA event
 * after every kernel on the context's work stream; ms_out[i] / launches_out[i]
 * receive the summed duration and launch count of kernel type i
 * (clover_profile_name(i)); nslots must be >= CLOVER_PROFILE_SLOTS. */
#define CLOVER_PROFILE_SLOTS 15
int clover_profile_steps(clover_ctx* ctx, int32_t nsteps, double* ms_out, int64_t* launches_out,
                         int32_t nslots);
const char* clover_profile_name(int32_t i);

/* Test: route every chunk boundary of a single-process multi-chunk context
 * through the remote-neighbour path (pack -> staging -> unpack, exactly the
 * code around the NCCL send/recv pair), so the multi-GPU message layout is
 * exercised on one GPU.  enable = 1: a device copy replaces the NCCL pair;
 * enable = 2: the messages travel through a one-rank NCCL communicator
 * (ncclSend/ncclRecv to self inside one group, created here) and dt through a
 * one-rank ncclAllReduce(MIN), captured in the step's CUDA graph like the
 * multi-rank path; enable = 3: as 2, but the messages are device-initiated
 * stores (S:8(f) f1): the pack kernel writes each message straight into its
 * receiver's slot of a one-rank NCCL symmetric window (ncclMemAlloc +
 * ncclCommWindowRegister, peer mapping from ncclGetPeerPointer), an LSA
 * barrier (ncclDevComm) makes the stores visible, the receiver unpacks, a
 * second barrier frees the mailbox -- the multi-rank path of CLOVER_LSA=1.
 * CLOVER_ERR_NCCL if the library was built without NCCL. */
int clover_debug_set_virtual_remote(clover_ctx* ctx, int32_t enable);

/* Debug: run only the first `nkernels` kernel phases of the next step
 * (1 = viscosity+calc_dt, 2 = +dt reduction, 3 = +Lagrangian phase,
 * 4..7 = +advection kernels); the step is left incomplete.  Test only. */
int clover_debug_partial_step(clover_ctx* ctx, int32_t nkernels);

/* Debug: read an internal buffer's global interior (ids as above plus
 * 100+ internal ids, see csrc/clover_engine.cu).  Test only. */
int clover_debug_read_buffer(clover_ctx* ctx, int32_t buffer_id, int32_t kind,
                             double* host, int64_t n);

/* Deep halos (S:8(f) f1): on y-strip layouts (px == 1,
 * py > 1, every chunk >= 16 rows, both fused sweeps) the state is exchanged
 * once per step, 7 rows deep, and each kernel of the step also computes the
 * rows of its y neighbours it would otherwise receive (visc_dt and the
 * Lagrangian phase 5 rows beyond each non-wall y side, sweep 1 4 (x) or 1
 * (y)), so a step has one halo exchange plus the dt MIN instead of three.
 * Results are bitwise identical either way.  enable = 1 / 0 (default 1, or
 * the environment's CLOVER_DEEP_HALO at clover_init); where the layout does
 * not qualify the setting has no effect.  clover_deep_halo_active reports
 * whether the next step uses it. */
int clover_set_deep_halo(clover_ctx* ctx, int32_t enable);
int clover_deep_halo_active(clover_ctx* ctx, int32_t* out);

/* Boundary-first overlap (S:8(e)): for y-strip layouts (px == 1) whose
 * exchanges take the remote path (several ranks, or virtual-remote mode),
 * each fused kernel runs the row segments next to a y chunk boundary first,
 * then the halo exchange on a second stream while the interior segments run;
 * the next kernel waits for both.  enable = 1 / 0 (default 0, or the
 * environment's CLOVER_OVERLAP at clover_init).  Results are bitwise
 * identical either way; tests compare them. */
int clover_debug_set_overlap(clover_ctx* ctx, int32_t enable);

/* Debug: the fused advection sweeps (advec_cell + advec_mom of one
 * direction in one pass).  enable = 1 (default): fused x sweep where every
 * local chunk has reflective walls on both x sides, fused y sweep everywhere
 * (at y chunk boundaries from depth-4 input halos); 2: fused y sweep only
 * where every chunk has both y walls (the separate kernels elsewhere); 0:
 * separate cell and momentum kernels throughout.  Geometric face mirror
 * only.  All settings are bitwise identical; tests compare them.  Test only. */
int clover_debug_set_fusion(clover_ctx* ctx, int32_t enable);

/* Debug: total number of warp segments the IEEE-division fixup launches
 * have recomputed since clover_init (DivFast flagged a numerator below
 * 2^-900 there), summed over local chunks.  Synchronises
 * the context's stream.  Test only. */
int clover_debug_fix_count(clover_ctx* ctx, int64_t* out);

/* Test: compare the library's internal fp64 division (div_rn) with IEEE
 * a/b bit for bit on n random operand pairs (exponents in [-emax, emax],
 * 1/16 zero numerators); *mismatches receives the count, example_ab (may be
 * NULL) the first mismatching pair.  Uses the current CUDA device. */
int clover_debug_div_check(int64_t n, uint64_t seed, int32_t emax, int64_t* mismatches,
                           double* example_ab);

/* ---- checkpoint / restart (sec. VI)
 * The library's access-execute description of one step (the reference's
 * loops with their read/write datasets) decides what a checkpoint must hold:
 * entering checkpoint mode before loop `loop` (0 = ideal_gas, i.e. the step
 * boundary ... 12 = reset_field), a dataset is saved iff its first access in
 * the periodic loop sequence is a read.  clover_checkpoint_plan returns that
 * set as a bit mask (bit order: density0, energy0, xvel0, yvel0, pressure,
 * soundspeed, viscosity, density1, energy1, xvel1, yvel1, vol_flux_x,
 * vol_flux_y, mass_flux_x, mass_flux_y), its size and the loop's name.
 * At the step boundary -- the optimum, where clover_checkpoint operates --
 * it is {density0, energy0, xvel0, yvel0}; plus the clock (step, time, dt,
 * dtold, sweep order).  Restarting from a checkpoint continues bit for bit.
 * Multi-rank: every rank gathers (and may write) the full checkpoint;
 * restart scatters each rank's part.  The buffer is host memory owned by the
 * caller. */
int clover_checkpoint_plan(int32_t loop, uint32_t* save_mask, int32_t* nsaved, const char** name);
int clover_checkpoint_bytes(clover_ctx* ctx, int64_t* bytes);
int clover_checkpoint(clover_ctx* ctx, void* host, int64_t bytes);
/* Restore a checkpoint taken on the same mesh (CLOVER_ERR_ARG otherwise). */
int clover_restart(clover_ctx* ctx, const void* host, int64_t bytes);

/* Destroy the context (does not free the caller's workspace). */
int clover_finalize(clover_ctx* ctx);

const char* clover_error_string(int code);
/* Last error message of this thread (argument validation details). */
const char* clover_last_error(void);
int clover_abi_version(void);

#ifdef __cplusplus
}
#endif
#endif /* CLOVER_H */
