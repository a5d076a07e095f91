/*
 * clover_oracle.h -- C API of the CPU ORACLE for the CloverLeaf 2D timestep.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and the
 * cpu_baseline / --impl reference legs of bench.py may load this library.
 * The product path (paper_conf_cluster_regulymg15_b200/) never includes,
 * links or calls anything under oracle/, and this file shares no code, header,
 * constant or helper with it.
 *
 * What it computes: one CloverLeaf 2D explicit Lagrangian-remap step of the
 * compressible Euler equations ("four partial differential equations ...
 * conservation of energy, density and momentum ... finite volume method on a
 * structured staggered grid", sec. V).  The paper states no
 * formulas; the arithmetic follows the reading written down in SURVEY.md
 * sec. 8(c) c.1-c.13 (public CloverLeaf 2D reference kernels), listed in
 * DESIGN.md "Readings".
 *
 * Index convention: j = x index, k = y index, 1-based
 * interior, logical halo depth 2.  Field read/write below use the GLOBAL
 * INTERIOR, row-major, j fastest: cells nx*ny, nodes (nx+1)*(ny+1),
 * x-faces (nx+1)*ny, y-faces nx*(ny+1).
 */
#ifndef CLOVER_ORACLE_H
#define CLOVER_ORACLE_H
#include <stdint.h>
#ifdef __cplusplus
extern "C" {
#endif

enum { OR_GEOM_RECT = 1, OR_GEOM_CIRCLE = 2, OR_GEOM_POINT = 3 };
/* A7 switch: how x-face fields are mirrored at bottom/top walls (and y-face
 * fields at left/right walls).  0 = geometric F(j,1-m)=F(j,m);
 * 1 = cell-centre F(j,1-m)=F(j,1+m), F(j,ny+m)=F(j,ny-m). */
enum { OR_MIRROR_GEOMETRIC = 0, OR_MIRROR_CELLCENTRE = 1 };

typedef struct {
  int32_t x_cells, y_cells;
  double xmin, ymin, xmax, ymax;
  double dtinit, dtmax, dtmin, dtrise;
  double dtc_safe, dtu_safe, dtv_safe, dtdiv_safe;
  int32_t advect_x_first; /* 1 = x sweep first on step 1 */
  int32_t face_mirror;    /* OR_MIRROR_* */
} oracle_grid;

typedef struct {
  double density, energy, xvel, yvel;
  int32_t geometry;
  double xmin, xmax, ymin, ymax, radius;
} oracle_state;

/* field ids */
enum {
  OF_DENSITY0 = 0, OF_ENERGY0, OF_PRESSURE, OF_VISCOSITY, OF_SOUNDSPEED,
  OF_XVEL0, OF_YVEL0, OF_DENSITY1, OF_ENERGY1, OF_XVEL1, OF_YVEL1,
  OF_VOL_FLUX_X, OF_VOL_FLUX_Y, OF_MASS_FLUX_X, OF_MASS_FLUX_Y, OF_NFIELDS
};

/* stage ids for oracle_run_stage (SURVEY 3(ii) hydro order) */
enum {
  OS_TIMESTEP = 0,  /* ideal_gas, halo, viscosity, halo, calc_dt, clamp */
  OS_PDV_PREDICT,   /* PdV(predict) + ideal_gas(predict) + halo{p} */
  OS_ACCELERATE,
  OS_PDV_CORRECT,
  OS_FLUX_CALC,
  OS_ADVECTION,     /* both sweeps */
  OS_RESET,         /* reset_field + advect_x flip + time/step */
  OS_ADV_CELL1,     /* advection() split into its four sub-steps, each with */
  OS_ADV_MOM1,      /* the halo updates that precede it in the reference   */
  OS_ADV_CELL2,
  OS_ADV_MOM2
};

typedef struct oracle_ctx oracle_ctx;

/* returns NULL on bad arguments */
oracle_ctx* oracle_create(const oracle_grid* g, const oracle_state* s, int32_t nstates);
void oracle_destroy(oracle_ctx* c);
/* run n full steps; dt_hist (may be NULL) receives n dts.
 * returns 0, or -5 if dt < dtmin (ref "small timestep"). */
int32_t oracle_step(oracle_ctx* c, int32_t n, double* dt_hist);
int32_t oracle_run_stage(oracle_ctx* c, int32_t stage);
/* field_summary: out = {vol, mass, ie, ke, press}, accumulated
 * sequentially in the reference's loop order (c.12). */
void oracle_field_summary(oracle_ctx* c, double* out5);
/* Same per-cell terms, accumulated with Neumaier compensated summation:
 * the totals to ~1 ulp, for meshes where the sequential sum's own rounding
 * (up to n*eps relative, 3e-9 at 3840^2) exceeds the 1e-10 parity gate. */
void oracle_field_summary_compensated(oracle_ctx* c, double* out5);
void oracle_clock(oracle_ctx* c, int32_t* step, double* time, double* dt, double* dtold);
int32_t oracle_read_field(oracle_ctx* c, int32_t fid, double* out, int64_t n);
/* writes the interior of a field; caller then calls oracle_refresh */
int32_t oracle_write_field(oracle_ctx* c, int32_t fid, const double* in, int64_t n);
/* start.f90 tail: ideal_gas(predict=F) + update_halo(all, depth 2) */
void oracle_refresh(oracle_ctx* c);

#ifdef __cplusplus
}
#endif
#endif
