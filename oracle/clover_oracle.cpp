/*
 * clover_oracle.cpp -- plain, slow, single-threaded CPU ORACLE of one
 * CloverLeaf 2D timestep (fp64).
 *
 * TEST INFRASTRUCTURE ONLY: loaded by tests/, __graft_entry__.smoke() and
 * bench.py's cpu_baseline / --impl reference legs, never by the product
 * path.  Shares no code with paper_conf_cluster_regulymg15_b200/.
 *
 * Source of the arithmetic.  PAPER.md:209 (sec. V) names the method only:
 * CloverLeaf 2D solves "the compressible Euler equations ... four partial
 * differential equations ... conservation of energy, density and momentum
 * ... finite volume method on a structured staggered grid".  The paper gives
 * no formulas, so every kernel below follows the reading in SURVEY.md
 * sec. 8(c) (c.1 ... c.13, the public CloverLeaf 2D v1.x reference kernels)
 * statement by statement, in the reference loop order, WITH the reference's
 * work arrays (pre_vol, post_vol, node_flux, ...) and halo-update calls, and
 * with Fortran left-to-right evaluation of same-precedence operators.
 * Build with -O2 -ffp-contract=off (no fast-math): no FMA contraction
 * (reading A8).
 *
 * Pins (tests/test_oracle_pins.py): closed forms P1/P2/P12, exact invariants
 * P3/P4/P4b/P7, mirror symmetry P5, exact Riemann solution P6, half-vs-
 * doubled domain P8, the recalled QA constant P10 (soft).  Every function
 * here is pinned by at least one of them.
 */
#include "clover_oracle.h"

#include <cmath>
#include <cstdlib>
#include <cstring>
#include <vector>
#include <algorithm>

namespace {

const double g_small = 1.0e-16;
const double g_big = 1.0e+21;
const double one_by_six = 1.0 / 6.0;

enum { XDIR = 1, YDIR = 2 };

/* A Fortran-style 2D array with index range j in [jlo, jhi], k in [klo, khi]. */
struct Arr {
  int jlo = 0, klo = 0, nj = 0, nk = 0;
  std::vector<double> v;
  void init(int jlo_, int jhi, int klo_, int khi) {
    jlo = jlo_; klo = klo_; nj = jhi - jlo_ + 1; nk = khi - klo_ + 1;
    v.assign((size_t)nj * nk, 0.0);
  }
  double& operator()(int j, int k) { return v[(size_t)(k - klo) * nj + (j - jlo)]; }
};

/* 1D array, index range [lo, hi] */
struct Vec {
  int lo = 0;
  std::vector<double> v;
  void init(int lo_, int hi) { lo = lo_; v.assign(hi - lo_ + 1, 0.0); }
  double& operator()(int j) { return v[j - lo]; }
};

enum FieldType { CELL, XVEL, YVEL, XFACE, YFACE };

}  // namespace

struct oracle_ctx {
  oracle_grid g;
  int x_min, x_max, y_min, y_max;
  double dx, dy;
  std::vector<oracle_state> states;
  /* fields */
  Arr density0, density1, energy0, energy1, pressure, viscosity, soundspeed;
  Arr xvel0, xvel1, yvel0, yvel1;
  Arr vol_flux_x, vol_flux_y, mass_flux_x, mass_flux_y;
  Arr volume, xarea, yarea;
  Arr work1, work2, work3, work4, work5, work6, work7;
  Vec cellx, celly, celldx, celldy, vertexx, vertexy, vertexdx, vertexdy;
  /* scalars (D7) */
  double dt, dtold, time;
  int step;
  bool advect_x;
};

namespace {

/* ------------------------------------------------------------------ */
/* c.10 update_halo: reflective boundary, physical faces only.         */
/* Order per field: bottom, top, left, right; each spans the full      */
/* other-axis extent including halos, so corners are double mirrors.   */
/* ------------------------------------------------------------------ */
void reflect(oracle_ctx* c, Arr& f, FieldType t, int depth) {
  const int x_min = c->x_min, x_max = c->x_max, y_min = c->y_min, y_max = c->y_max;
  const bool geo = c->g.face_mirror == OR_MIRROR_GEOMETRIC;
  switch (t) {
    case CELL:
      for (int j = x_min - depth; j <= x_max + depth; ++j)
        for (int k = 1; k <= depth; ++k) f(j, 1 - k) = f(j, 0 + k);
      for (int j = x_min - depth; j <= x_max + depth; ++j)
        for (int k = 1; k <= depth; ++k) f(j, y_max + k) = f(j, y_max + 1 - k);
      for (int k = y_min - depth; k <= y_max + depth; ++k)
        for (int j = 1; j <= depth; ++j) f(1 - j, k) = f(0 + j, k);
      for (int k = y_min - depth; k <= y_max + depth; ++k)
        for (int j = 1; j <= depth; ++j) f(x_max + j, k) = f(x_max + 1 - j, k);
      break;
    case XVEL:
      for (int j = x_min - depth; j <= x_max + 1 + depth; ++j)
        for (int k = 1; k <= depth; ++k) f(j, 1 - k) = f(j, 1 + k);
      for (int j = x_min - depth; j <= x_max + 1 + depth; ++j)
        for (int k = 1; k <= depth; ++k) f(j, y_max + 1 + k) = f(j, y_max + 1 - k);
      for (int k = y_min - depth; k <= y_max + 1 + depth; ++k)
        for (int j = 1; j <= depth; ++j) f(1 - j, k) = -f(1 + j, k);
      for (int k = y_min - depth; k <= y_max + 1 + depth; ++k)
        for (int j = 1; j <= depth; ++j) f(x_max + 1 + j, k) = -f(x_max + 1 - j, k);
      break;
    case YVEL:
      for (int j = x_min - depth; j <= x_max + 1 + depth; ++j)
        for (int k = 1; k <= depth; ++k) f(j, 1 - k) = -f(j, 1 + k);
      for (int j = x_min - depth; j <= x_max + 1 + depth; ++j)
        for (int k = 1; k <= depth; ++k) f(j, y_max + 1 + k) = -f(j, y_max + 1 - k);
      for (int k = y_min - depth; k <= y_max + 1 + depth; ++k)
        for (int j = 1; j <= depth; ++j) f(1 - j, k) = f(1 + j, k);
      for (int k = y_min - depth; k <= y_max + 1 + depth; ++k)
        for (int j = 1; j <= depth; ++j) f(x_max + 1 + j, k) = f(x_max + 1 - j, k);
      break;
    case XFACE: /* tangential (y) mirror: reading A7 */
      for (int j = x_min - depth; j <= x_max + 1 + depth; ++j)
        for (int k = 1; k <= depth; ++k) f(j, 1 - k) = geo ? f(j, k) : f(j, 1 + k);
      for (int j = x_min - depth; j <= x_max + 1 + depth; ++j)
        for (int k = 1; k <= depth; ++k)
          f(j, y_max + k) = geo ? f(j, y_max + 1 - k) : f(j, y_max - k);
      for (int k = y_min - depth; k <= y_max + depth; ++k)
        for (int j = 1; j <= depth; ++j) f(1 - j, k) = -f(1 + j, k);
      for (int k = y_min - depth; k <= y_max + depth; ++k)
        for (int j = 1; j <= depth; ++j) f(x_max + 1 + j, k) = -f(x_max + 1 - j, k);
      break;
    case YFACE:
      for (int j = x_min - depth; j <= x_max + depth; ++j)
        for (int k = 1; k <= depth; ++k) f(j, 1 - k) = -f(j, 1 + k);
      for (int j = x_min - depth; j <= x_max + depth; ++j)
        for (int k = 1; k <= depth; ++k) f(j, y_max + 1 + k) = -f(j, y_max + 1 - k);
      for (int k = y_min - depth; k <= y_max + 1 + depth; ++k)  /* tangential (x): A7 */
        for (int j = 1; j <= depth; ++j) f(1 - j, k) = geo ? f(j, k) : f(1 + j, k);
      for (int k = y_min - depth; k <= y_max + 1 + depth; ++k)
        for (int j = 1; j <= depth; ++j)
          f(x_max + j, k) = geo ? f(x_max + 1 - j, k) : f(x_max - j, k);
      break;
  }
}

/* c.2 ideal_gas (interior cells) */
void ideal_gas(oracle_ctx* c, bool predict) {
  Arr& density = predict ? c->density1 : c->density0;
  Arr& energy = predict ? c->energy1 : c->energy0;
  const double gm1 = 1.4 - 1.0; /* reading A2: evaluated in fp64 */
  for (int k = c->y_min; k <= c->y_max; ++k)
    for (int j = c->x_min; j <= c->x_max; ++j) {
      double v = 1.0 / density(j, k);
      c->pressure(j, k) = gm1 * density(j, k) * energy(j, k);
      double pressurebyenergy = gm1 * density(j, k);
      double pressurebyvolume = -density(j, k) * c->pressure(j, k);
      double sound_speed_squared = v * v * (c->pressure(j, k) * pressurebyenergy - pressurebyvolume);
      c->soundspeed(j, k) = std::sqrt(sound_speed_squared);
    }
}

/* c.3 viscosity */
void viscosity(oracle_ctx* c) {
  Arr& u = c->xvel0; Arr& v = c->yvel0; Arr& p = c->pressure;
  for (int k = c->y_min; k <= c->y_max; ++k)
    for (int j = c->x_min; j <= c->x_max; ++j) {
      double ugrad = (u(j + 1, k) + u(j + 1, k + 1)) - (u(j, k) + u(j, k + 1));
      double vgrad = (v(j, k + 1) + v(j + 1, k + 1)) - (v(j, k) + v(j + 1, k));
      double div = (c->celldx(j) * (ugrad) + c->celldy(k) * (vgrad));
      double strain2 = 0.5 * (u(j, k + 1) + u(j + 1, k + 1) - u(j, k) - u(j + 1, k)) / c->celldy(k)
                     + 0.5 * (v(j + 1, k) + v(j + 1, k + 1) - v(j, k) - v(j, k + 1)) / c->celldx(j);
      double pgradx = (p(j + 1, k) - p(j - 1, k)) / (c->celldx(j) + c->celldx(j + 1));
      double pgrady = (p(j, k + 1) - p(j, k - 1)) / (c->celldy(k) + c->celldy(k + 1));
      double pgradx2 = pgradx * pgradx;
      double pgrady2 = pgrady * pgrady;
      double limiter = ((0.5 * (ugrad) / c->celldx(j)) * pgradx2
                        + (0.5 * (vgrad) / c->celldy(k)) * pgrady2
                        + strain2 * pgradx * pgrady)
                       / std::max(pgradx2 + pgrady2, 1.0e-16);
      if ((limiter > 0.0) || (div >= 0.0)) {
        c->viscosity(j, k) = 0.0;
      } else {
        pgradx = std::copysign(std::max(1.0e-16, std::fabs(pgradx)), pgradx);
        pgrady = std::copysign(std::max(1.0e-16, std::fabs(pgrady)), pgrady);
        double pgrad = std::sqrt(pgradx * pgradx + pgrady * pgrady);
        double xgrad = std::fabs(c->celldx(j) * pgrad / pgradx);
        double ygrad = std::fabs(c->celldy(k) * pgrad / pgrady);
        double grad = std::min(xgrad, ygrad);
        double grad2 = grad * grad;
        c->viscosity(j, k) = 2.0 * c->density0(j, k) * grad2 * limiter * limiter;
      }
    }
}

/* c.4 calc_dt kernel: minimum over interior cells */
double calc_dt(oracle_ctx* c) {
  double dt_min_val = g_big;
  const oracle_grid& g = c->g;
  for (int k = c->y_min; k <= c->y_max; ++k)
    for (int j = c->x_min; j <= c->x_max; ++j) {
      double dsx = c->celldx(j);
      double dsy = c->celldy(k);
      double cc = c->soundspeed(j, k) * c->soundspeed(j, k);
      cc = cc + 2.0 * c->viscosity(j, k) / c->density0(j, k);
      cc = std::max(std::sqrt(cc), g_small);
      double dtct = g.dtc_safe * std::min(dsx, dsy) / cc;
      double div = 0.0;
      double dv1 = (c->xvel0(j, k) + c->xvel0(j, k + 1)) * c->xarea(j, k);
      double dv2 = (c->xvel0(j + 1, k) + c->xvel0(j + 1, k + 1)) * c->xarea(j + 1, k);
      div = div + dv2 - dv1;
      double dtut = g.dtu_safe * 2.0 * c->volume(j, k)
                    / std::max(std::max(std::fabs(dv1), std::fabs(dv2)), g_small * c->volume(j, k));
      dv1 = (c->yvel0(j, k) + c->yvel0(j + 1, k)) * c->yarea(j, k);
      dv2 = (c->yvel0(j, k + 1) + c->yvel0(j + 1, k + 1)) * c->yarea(j, k + 1);
      div = div + dv2 - dv1;
      double dtvt = g.dtv_safe * 2.0 * c->volume(j, k)
                    / std::max(std::max(std::fabs(dv1), std::fabs(dv2)), g_small * c->volume(j, k));
      div = div / (2.0 * c->volume(j, k));
      double dtdivt;
      if (div < -g_small)
        dtdivt = g.dtdiv_safe * (-1.0 / div);
      else
        dtdivt = g_big;
      dt_min_val = std::min(dt_min_val, std::min(std::min(dtct, dtut), std::min(dtvt, dtdivt)));
    }
  return dt_min_val;
}

/* c.5 PdV */
void pdv(oracle_ctx* c, bool predict) {
  const double dt = c->dt;
  Arr& xv0 = c->xvel0; Arr& yv0 = c->yvel0; Arr& xv1 = c->xvel1; Arr& yv1 = c->yvel1;
  Arr& volume_change = c->work1;
  for (int k = c->y_min; k <= c->y_max; ++k)
    for (int j = c->x_min; j <= c->x_max; ++j) {
      double left_flux, right_flux, bottom_flux, top_flux;
      if (predict) {
        left_flux = (c->xarea(j, k) * (xv0(j, k) + xv0(j, k + 1) + xv0(j, k) + xv0(j, k + 1))) * 0.25 * dt * 0.5;
        right_flux = (c->xarea(j + 1, k) * (xv0(j + 1, k) + xv0(j + 1, k + 1) + xv0(j + 1, k) + xv0(j + 1, k + 1))) * 0.25 * dt * 0.5;
        bottom_flux = (c->yarea(j, k) * (yv0(j, k) + yv0(j + 1, k) + yv0(j, k) + yv0(j + 1, k))) * 0.25 * dt * 0.5;
        top_flux = (c->yarea(j, k + 1) * (yv0(j, k + 1) + yv0(j + 1, k + 1) + yv0(j, k + 1) + yv0(j + 1, k + 1))) * 0.25 * dt * 0.5;
      } else {
        left_flux = (c->xarea(j, k) * (xv0(j, k) + xv0(j, k + 1) + xv1(j, k) + xv1(j, k + 1))) * 0.25 * dt;
        right_flux = (c->xarea(j + 1, k) * (xv0(j + 1, k) + xv0(j + 1, k + 1) + xv1(j + 1, k) + xv1(j + 1, k + 1))) * 0.25 * dt;
        bottom_flux = (c->yarea(j, k) * (yv0(j, k) + yv0(j + 1, k) + yv1(j, k) + yv1(j + 1, k))) * 0.25 * dt;
        top_flux = (c->yarea(j, k + 1) * (yv0(j, k + 1) + yv0(j + 1, k + 1) + yv1(j, k + 1) + yv1(j + 1, k + 1))) * 0.25 * dt;
      }
      double total_flux = right_flux - left_flux + top_flux - bottom_flux;
      volume_change(j, k) = c->volume(j, k) / (c->volume(j, k) + total_flux);
      double recip_volume = 1.0 / c->volume(j, k);
      double energy_change = (c->pressure(j, k) / c->density0(j, k) + c->viscosity(j, k) / c->density0(j, k))
                             * total_flux * recip_volume;
      c->energy1(j, k) = c->energy0(j, k) - energy_change;
      c->density1(j, k) = c->density0(j, k) * volume_change(j, k);
    }
}

/* c.6 accelerate (nodes x_min..x_max+1, y_min..y_max+1) */
void accelerate(oracle_ctx* c) {
  const double halfdt = 0.5 * c->dt;
  Arr& stepbymass = c->work1;
  Arr& d0 = c->density0; Arr& vol = c->volume; Arr& p = c->pressure; Arr& q = c->viscosity;
  for (int k = c->y_min; k <= c->y_max + 1; ++k)
    for (int j = c->x_min; j <= c->x_max + 1; ++j) {
      double nodal_mass = (d0(j - 1, k - 1) * vol(j - 1, k - 1) + d0(j, k - 1) * vol(j, k - 1)
                           + d0(j, k) * vol(j, k) + d0(j - 1, k) * vol(j - 1, k)) * 0.25;
      stepbymass(j, k) = halfdt / nodal_mass;
    }
  for (int k = c->y_min; k <= c->y_max + 1; ++k)
    for (int j = c->x_min; j <= c->x_max + 1; ++j) {
      c->xvel1(j, k) = c->xvel0(j, k) - stepbymass(j, k) * (c->xarea(j, k) * (p(j, k) - p(j - 1, k))
                                                           + c->xarea(j, k - 1) * (p(j, k - 1) - p(j - 1, k - 1)));
      c->yvel1(j, k) = c->yvel0(j, k) - stepbymass(j, k) * (c->yarea(j, k) * (p(j, k) - p(j, k - 1))
                                                           + c->yarea(j - 1, k) * (p(j - 1, k) - p(j - 1, k - 1)));
    }
  for (int k = c->y_min; k <= c->y_max + 1; ++k)
    for (int j = c->x_min; j <= c->x_max + 1; ++j) {
      c->xvel1(j, k) = c->xvel1(j, k) - stepbymass(j, k) * (c->xarea(j, k) * (q(j, k) - q(j - 1, k))
                                                           + c->xarea(j, k - 1) * (q(j, k - 1) - q(j - 1, k - 1)));
      c->yvel1(j, k) = c->yvel1(j, k) - stepbymass(j, k) * (c->yarea(j, k) * (q(j, k) - q(j, k - 1))
                                                           + c->yarea(j - 1, k) * (q(j - 1, k) - q(j - 1, k - 1)));
    }
}

/* c.7 flux_calc */
void flux_calc(oracle_ctx* c) {
  const double dt = c->dt;
  for (int k = c->y_min; k <= c->y_max; ++k)
    for (int j = c->x_min; j <= c->x_max + 1; ++j)
      c->vol_flux_x(j, k) = 0.25 * dt * c->xarea(j, k)
                            * (c->xvel0(j, k) + c->xvel0(j, k + 1) + c->xvel1(j, k) + c->xvel1(j, k + 1));
  for (int k = c->y_min; k <= c->y_max + 1; ++k)
    for (int j = c->x_min; j <= c->x_max; ++j)
      c->vol_flux_y(j, k) = 0.25 * dt * c->yarea(j, k)
                            * (c->yvel0(j, k) + c->yvel0(j + 1, k) + c->yvel1(j, k) + c->yvel1(j + 1, k));
}

/* c.8 advec_cell */
void advec_cell(oracle_ctx* c, int dir, int sweep_number) {
  const int x_min = c->x_min, x_max = c->x_max, y_min = c->y_min, y_max = c->y_max;
  Arr& pre_vol = c->work1; Arr& post_vol = c->work2; Arr& pre_mass = c->work3;
  Arr& post_mass = c->work4; Arr& advec_vol = c->work5; Arr& post_ener = c->work6;
  Arr& ener_flux = c->work7;
  Arr& vfx = c->vol_flux_x; Arr& vfy = c->vol_flux_y;
  Arr& d1 = c->density1; Arr& e1 = c->energy1; Arr& vol = c->volume;
  if (dir == XDIR) {
    if (sweep_number == 1) {
      for (int k = y_min - 2; k <= y_max + 2; ++k)
        for (int j = x_min - 2; j <= x_max + 2; ++j) {
          pre_vol(j, k) = vol(j, k) + (vfx(j + 1, k) - vfx(j, k) + vfy(j, k + 1) - vfy(j, k));
          post_vol(j, k) = pre_vol(j, k) - (vfx(j + 1, k) - vfx(j, k));
        }
    } else {
      for (int k = y_min - 2; k <= y_max + 2; ++k)
        for (int j = x_min - 2; j <= x_max + 2; ++j) {
          pre_vol(j, k) = vol(j, k) + vfx(j + 1, k) - vfx(j, k);
          post_vol(j, k) = vol(j, k);
        }
    }
    Arr& mfx = c->mass_flux_x;
    for (int k = y_min; k <= y_max; ++k)
      for (int j = x_min; j <= x_max + 2; ++j) {
        int upwind, donor, downwind, dif;
        if (vfx(j, k) > 0.0) {
          upwind = j - 2; donor = j - 1; downwind = j; dif = donor;
        } else {
          upwind = std::min(j + 1, x_max + 2); donor = j; downwind = j - 1; dif = upwind;
        }
        double sigmat = std::fabs(vfx(j, k)) / pre_vol(donor, k);
        double sigma3 = (1.0 + sigmat) * (c->vertexdx(j) / c->vertexdx(dif));
        double sigma4 = 2.0 - sigmat;
        double sigmav = sigmat;
        double diffuw = d1(donor, k) - d1(upwind, k);
        double diffdw = d1(downwind, k) - d1(donor, k);
        double wind = 1.0;
        if (diffdw <= 0.0) wind = -1.0;
        double limiter;
        if (diffuw * diffdw > 0.0)
          limiter = (1.0 - sigmav) * wind
                    * std::min(std::min(std::fabs(diffuw), std::fabs(diffdw)),
                               one_by_six * (sigma3 * std::fabs(diffuw) + sigma4 * std::fabs(diffdw)));
        else
          limiter = 0.0;
        mfx(j, k) = vfx(j, k) * (d1(donor, k) + limiter);
        double sigmam = std::fabs(mfx(j, k)) / (d1(donor, k) * pre_vol(donor, k));
        diffuw = e1(donor, k) - e1(upwind, k);
        diffdw = e1(downwind, k) - e1(donor, k);
        wind = 1.0;
        if (diffdw <= 0.0) wind = -1.0;
        if (diffuw * diffdw > 0.0)
          limiter = (1.0 - sigmam) * wind
                    * std::min(std::min(std::fabs(diffuw), std::fabs(diffdw)),
                               one_by_six * (sigma3 * std::fabs(diffuw) + sigma4 * std::fabs(diffdw)));
        else
          limiter = 0.0;
        ener_flux(j, k) = mfx(j, k) * (e1(donor, k) + limiter);
      }
    for (int k = y_min; k <= y_max; ++k)
      for (int j = x_min; j <= x_max; ++j) {
        pre_mass(j, k) = d1(j, k) * pre_vol(j, k);
        post_mass(j, k) = pre_mass(j, k) + mfx(j, k) - mfx(j + 1, k);
        post_ener(j, k) = (e1(j, k) * pre_mass(j, k) + ener_flux(j, k) - ener_flux(j + 1, k)) / post_mass(j, k);
        advec_vol(j, k) = pre_vol(j, k) + vfx(j, k) - vfx(j + 1, k);
        d1(j, k) = post_mass(j, k) / advec_vol(j, k);
        e1(j, k) = post_ener(j, k);
      }
  } else {
    if (sweep_number == 1) {
      for (int k = y_min - 2; k <= y_max + 2; ++k)
        for (int j = x_min - 2; j <= x_max + 2; ++j) {
          pre_vol(j, k) = vol(j, k) + (vfy(j, k + 1) - vfy(j, k) + vfx(j + 1, k) - vfx(j, k));
          post_vol(j, k) = pre_vol(j, k) - (vfy(j, k + 1) - vfy(j, k));
        }
    } else {
      for (int k = y_min - 2; k <= y_max + 2; ++k)
        for (int j = x_min - 2; j <= x_max + 2; ++j) {
          pre_vol(j, k) = vol(j, k) + vfy(j, k + 1) - vfy(j, k);
          post_vol(j, k) = vol(j, k);
        }
    }
    Arr& mfy = c->mass_flux_y;
    for (int k = y_min; k <= y_max + 2; ++k)
      for (int j = x_min; j <= x_max; ++j) {
        int upwind, donor, downwind, dif;
        if (vfy(j, k) > 0.0) {
          upwind = k - 2; donor = k - 1; downwind = k; dif = donor;
        } else {
          upwind = std::min(k + 1, y_max + 2); donor = k; downwind = k - 1; dif = upwind;
        }
        double sigmat = std::fabs(vfy(j, k)) / pre_vol(j, donor);
        double sigma3 = (1.0 + sigmat) * (c->vertexdy(k) / c->vertexdy(dif));
        double sigma4 = 2.0 - sigmat;
        double sigmav = sigmat;
        double diffuw = d1(j, donor) - d1(j, upwind);
        double diffdw = d1(j, downwind) - d1(j, donor);
        double wind = 1.0;
        if (diffdw <= 0.0) wind = -1.0;
        double limiter;
        if (diffuw * diffdw > 0.0)
          limiter = (1.0 - sigmav) * wind
                    * std::min(std::min(std::fabs(diffuw), std::fabs(diffdw)),
                               one_by_six * (sigma3 * std::fabs(diffuw) + sigma4 * std::fabs(diffdw)));
        else
          limiter = 0.0;
        mfy(j, k) = vfy(j, k) * (d1(j, donor) + limiter);
        double sigmam = std::fabs(mfy(j, k)) / (d1(j, donor) * pre_vol(j, donor));
        diffuw = e1(j, donor) - e1(j, upwind);
        diffdw = e1(j, downwind) - e1(j, donor);
        wind = 1.0;
        if (diffdw <= 0.0) wind = -1.0;
        if (diffuw * diffdw > 0.0)
          limiter = (1.0 - sigmam) * wind
                    * std::min(std::min(std::fabs(diffuw), std::fabs(diffdw)),
                               one_by_six * (sigma3 * std::fabs(diffuw) + sigma4 * std::fabs(diffdw)));
        else
          limiter = 0.0;
        ener_flux(j, k) = mfy(j, k) * (e1(j, donor) + limiter);
      }
    for (int k = y_min; k <= y_max; ++k)
      for (int j = x_min; j <= x_max; ++j) {
        pre_mass(j, k) = d1(j, k) * pre_vol(j, k);
        post_mass(j, k) = pre_mass(j, k) + mfy(j, k) - mfy(j, k + 1);
        post_ener(j, k) = (e1(j, k) * pre_mass(j, k) + ener_flux(j, k) - ener_flux(j, k + 1)) / post_mass(j, k);
        advec_vol(j, k) = pre_vol(j, k) + vfy(j, k) - vfy(j, k + 1);
        d1(j, k) = post_mass(j, k) / advec_vol(j, k);
        e1(j, k) = post_ener(j, k);
      }
  }
}

/* c.9 advec_mom; which_vel 1 = xvel1 (computes the node quantities),
 * 2 = yvel1 (reuses them, as the reference does) */
void advec_mom(oracle_ctx* c, int which_vel, int direction, int sweep_number) {
  const int x_min = c->x_min, x_max = c->x_max, y_min = c->y_min, y_max = c->y_max;
  Arr& vel1 = which_vel == 1 ? c->xvel1 : c->yvel1;
  Arr& node_flux = c->work1; Arr& node_mass_post = c->work2; Arr& node_mass_pre = c->work3;
  Arr& advec_vel = c->work4; Arr& mom_flux = c->work5; Arr& pre_vol = c->work6; Arr& post_vol = c->work7;
  Arr& vfx = c->vol_flux_x; Arr& vfy = c->vol_flux_y; Arr& vol = c->volume; Arr& d1 = c->density1;
  int mom_sweep = direction + 2 * (sweep_number - 1);
  if (mom_sweep == 1) {        /* x 1 */
    for (int k = y_min - 2; k <= y_max + 2; ++k)
      for (int j = x_min - 2; j <= x_max + 2; ++j) {
        post_vol(j, k) = vol(j, k) + vfy(j, k + 1) - vfy(j, k);
        pre_vol(j, k) = post_vol(j, k) + vfx(j + 1, k) - vfx(j, k);
      }
  } else if (mom_sweep == 2) { /* y 1 */
    for (int k = y_min - 2; k <= y_max + 2; ++k)
      for (int j = x_min - 2; j <= x_max + 2; ++j) {
        post_vol(j, k) = vol(j, k) + vfx(j + 1, k) - vfx(j, k);
        pre_vol(j, k) = post_vol(j, k) + vfy(j, k + 1) - vfy(j, k);
      }
  } else if (mom_sweep == 3) { /* x 2 */
    for (int k = y_min - 2; k <= y_max + 2; ++k)
      for (int j = x_min - 2; j <= x_max + 2; ++j) {
        post_vol(j, k) = vol(j, k);
        pre_vol(j, k) = post_vol(j, k) + vfy(j, k + 1) - vfy(j, k);
      }
  } else {                     /* y 2 */
    for (int k = y_min - 2; k <= y_max + 2; ++k)
      for (int j = x_min - 2; j <= x_max + 2; ++j) {
        post_vol(j, k) = vol(j, k);
        pre_vol(j, k) = post_vol(j, k) + vfx(j + 1, k) - vfx(j, k);
      }
  }
  if (direction == XDIR) {
    Arr& mfx = c->mass_flux_x;
    if (which_vel == 1) {
      for (int k = y_min; k <= y_max + 1; ++k)
        for (int j = x_min - 2; j <= x_max + 2; ++j)
          node_flux(j, k) = 0.25 * (mfx(j, k - 1) + mfx(j, k) + mfx(j + 1, k - 1) + mfx(j + 1, k));
      for (int k = y_min; k <= y_max + 1; ++k)
        for (int j = x_min - 1; j <= x_max + 2; ++j) {
          node_mass_post(j, k) = 0.25 * (d1(j, k - 1) * post_vol(j, k - 1) + d1(j, k) * post_vol(j, k)
                                         + d1(j - 1, k - 1) * post_vol(j - 1, k - 1)
                                         + d1(j - 1, k) * post_vol(j - 1, k));
          node_mass_pre(j, k) = node_mass_post(j, k) - node_flux(j - 1, k) + node_flux(j, k);
        }
    }
    for (int k = y_min; k <= y_max + 1; ++k)
      for (int j = x_min - 1; j <= x_max + 1; ++j) {
        int upwind, donor, downwind, dif;
        if (node_flux(j, k) < 0.0) {
          upwind = j + 2; donor = j + 1; downwind = j; dif = donor;
        } else {
          upwind = j - 1; donor = j; downwind = j + 1; dif = upwind;
        }
        double sigma = std::fabs(node_flux(j, k)) / (node_mass_pre(donor, k));
        double width = c->celldx(j);
        double vdiffuw = vel1(donor, k) - vel1(upwind, k);
        double vdiffdw = vel1(downwind, k) - vel1(donor, k);
        double limiter = 0.0;
        if (vdiffuw * vdiffdw > 0.0) {
          double auw = std::fabs(vdiffuw);
          double adw = std::fabs(vdiffdw);
          double wind = 1.0;
          if (vdiffdw <= 0.0) wind = -1.0;
          limiter = wind * std::min(std::min(width * ((2.0 - sigma) * adw / width
                                                      + (1.0 + sigma) * auw / c->celldx(dif)) / 6.0,
                                             auw), adw);
        }
        advec_vel(j, k) = vel1(donor, k) + (1.0 - sigma) * limiter;
        mom_flux(j, k) = advec_vel(j, k) * node_flux(j, k);
      }
    for (int k = y_min; k <= y_max + 1; ++k)
      for (int j = x_min; j <= x_max + 1; ++j)
        vel1(j, k) = (vel1(j, k) * node_mass_pre(j, k) + mom_flux(j - 1, k) - mom_flux(j, k)) / node_mass_post(j, k);
  } else {
    Arr& mfy = c->mass_flux_y;
    if (which_vel == 1) {
      for (int k = y_min - 2; k <= y_max + 2; ++k)
        for (int j = x_min; j <= x_max + 1; ++j)
          node_flux(j, k) = 0.25 * (mfy(j - 1, k) + mfy(j, k) + mfy(j - 1, k + 1) + mfy(j, k + 1));
      for (int k = y_min - 1; k <= y_max + 2; ++k)
        for (int j = x_min; j <= x_max + 1; ++j) {
          node_mass_post(j, k) = 0.25 * (d1(j, k - 1) * post_vol(j, k - 1) + d1(j, k) * post_vol(j, k)
                                         + d1(j - 1, k - 1) * post_vol(j - 1, k - 1)
                                         + d1(j - 1, k) * post_vol(j - 1, k));
          node_mass_pre(j, k) = node_mass_post(j, k) - node_flux(j, k - 1) + node_flux(j, k);
        }
    }
    for (int k = y_min - 1; k <= y_max + 1; ++k)
      for (int j = x_min; j <= x_max + 1; ++j) {
        int upwind, donor, downwind, dif;
        if (node_flux(j, k) < 0.0) {
          upwind = k + 2; donor = k + 1; downwind = k; dif = donor;
        } else {
          upwind = k - 1; donor = k; downwind = k + 1; dif = upwind;
        }
        double sigma = std::fabs(node_flux(j, k)) / (node_mass_pre(j, donor));
        double width = c->celldy(k);
        double vdiffuw = vel1(j, donor) - vel1(j, upwind);
        double vdiffdw = vel1(j, downwind) - vel1(j, donor);
        double limiter = 0.0;
        if (vdiffuw * vdiffdw > 0.0) {
          double auw = std::fabs(vdiffuw);
          double adw = std::fabs(vdiffdw);
          double wind = 1.0;
          if (vdiffdw <= 0.0) wind = -1.0;
          limiter = wind * std::min(std::min(width * ((2.0 - sigma) * adw / width
                                                      + (1.0 + sigma) * auw / c->celldy(dif)) / 6.0,
                                             auw), adw);
        }
        advec_vel(j, k) = vel1(j, donor) + (1.0 - sigma) * limiter;
        mom_flux(j, k) = advec_vel(j, k) * node_flux(j, k);
      }
    for (int k = y_min; k <= y_max + 1; ++k)
      for (int j = x_min; j <= x_max + 1; ++j)
        vel1(j, k) = (vel1(j, k) * node_mass_pre(j, k) + mom_flux(j, k - 1) - mom_flux(j, k)) / node_mass_post(j, k);
  }
}

/* SURVEY 3(ii) timestep(): EOS, halo, viscosity, halo, calc_dt, clamp */
int timestep(oracle_ctx* c) {
  ideal_gas(c, false);
  reflect(c, c->pressure, CELL, 1);
  reflect(c, c->energy0, CELL, 1);
  reflect(c, c->density0, CELL, 1);
  reflect(c, c->xvel0, XVEL, 1);
  reflect(c, c->yvel0, YVEL, 1);
  viscosity(c);
  reflect(c, c->viscosity, CELL, 1);
  double dt = calc_dt(c);
  dt = std::min(std::min(dt, (c->dtold * c->g.dtrise)), c->g.dtmax);
  c->dt = dt;
  if (dt < c->g.dtmin) return -5;
  c->dtold = dt;
  return 0;
}

/* advection() of SURVEY 3(ii), split into its sub-steps so tests can stop
 * between them; advection() runs all four in order. */
void advection_part(oracle_ctx* c, int part) {
  const int d1 = c->advect_x ? XDIR : YDIR;
  const int d2 = c->advect_x ? YDIR : XDIR;
  if (part == 0) {
    reflect(c, c->energy1, CELL, 2);
    reflect(c, c->density1, CELL, 2);
    reflect(c, c->vol_flux_x, XFACE, 2);
    reflect(c, c->vol_flux_y, YFACE, 2);
    advec_cell(c, d1, 1);
  } else if (part == 1 || part == 3) {
    reflect(c, c->density1, CELL, 2);
    reflect(c, c->energy1, CELL, 2);
    reflect(c, c->xvel1, XVEL, 2);
    reflect(c, c->yvel1, YVEL, 2);
    reflect(c, c->mass_flux_x, XFACE, 2);
    reflect(c, c->mass_flux_y, YFACE, 2);
    const int d = part == 1 ? d1 : d2;
    const int sweep = part == 1 ? 1 : 2;
    advec_mom(c, 1, d, sweep);
    advec_mom(c, 2, d, sweep);
  } else {
    advec_cell(c, d2, 2);
  }
}

void advection(oracle_ctx* c) {
  for (int part = 0; part < 4; ++part) advection_part(c, part);
}

/* c.11 reset_field */
void reset_field(oracle_ctx* c) {
  for (int k = c->y_min; k <= c->y_max; ++k)
    for (int j = c->x_min; j <= c->x_max; ++j) {
      c->density0(j, k) = c->density1(j, k);
      c->energy0(j, k) = c->energy1(j, k);
    }
  for (int k = c->y_min; k <= c->y_max + 1; ++k)
    for (int j = c->x_min; j <= c->x_max + 1; ++j) {
      c->xvel0(j, k) = c->xvel1(j, k);
      c->yvel0(j, k) = c->yvel1(j, k);
    }
}

void pdv_predict_stage(oracle_ctx* c) {
  pdv(c, true);
  ideal_gas(c, true);
  reflect(c, c->pressure, CELL, 1);
  /* revert (density1=density0, energy1=energy0) is skipped: the corrector
   * overwrites density1/energy1 on every cell that is read (reading A11). */
}

void finish_step(oracle_ctx* c) {
  reset_field(c);
  c->advect_x = !c->advect_x;
  c->time = c->time + c->dt;
  c->step += 1;
}

int full_step(oracle_ctx* c) {
  int rc = timestep(c);
  if (rc) return rc;
  pdv_predict_stage(c);
  accelerate(c);
  pdv(c, false);
  flux_calc(c);
  advection(c);
  finish_step(c);
  return 0;
}

/* c.1 initialise_chunk + generate_chunk */
void initialise(oracle_ctx* c) {
  const int nx = c->g.x_cells, ny = c->g.y_cells;
  c->x_min = 1; c->x_max = nx; c->y_min = 1; c->y_max = ny;
  Arr* all[] = {&c->density0, &c->density1, &c->energy0, &c->energy1, &c->pressure, &c->viscosity,
                &c->soundspeed, &c->xvel0, &c->xvel1, &c->yvel0, &c->yvel1, &c->vol_flux_x,
                &c->vol_flux_y, &c->mass_flux_x, &c->mass_flux_y, &c->volume, &c->xarea, &c->yarea,
                &c->work1, &c->work2, &c->work3, &c->work4, &c->work5, &c->work6, &c->work7};
  for (Arr* a : all) a->init(-1, nx + 3, -1, ny + 3);  /* node-sized, halo depth 2 */
  Vec* vecs[] = {&c->cellx, &c->celly, &c->celldx, &c->celldy, &c->vertexx, &c->vertexy,
                 &c->vertexdx, &c->vertexdy};
  for (Vec* v : vecs) v->init(-1, std::max(nx, ny) + 3);

  /* geometry from the GLOBAL index (reading A13) */
  double dx = (c->g.xmax - c->g.xmin) / (double)nx;
  double dy = (c->g.ymax - c->g.ymin) / (double)ny;
  c->dx = dx; c->dy = dy;
  for (int j = -1; j <= nx + 3; ++j) { c->vertexx(j) = c->g.xmin + dx * (double)(j - 1); c->vertexdx(j) = dx; }
  for (int k = -1; k <= ny + 3; ++k) { c->vertexy(k) = c->g.ymin + dy * (double)(k - 1); c->vertexdy(k) = dy; }
  for (int j = -1; j <= nx + 2; ++j) { c->cellx(j) = 0.5 * (c->vertexx(j) + c->vertexx(j + 1)); c->celldx(j) = dx; }
  for (int k = -1; k <= ny + 2; ++k) { c->celly(k) = 0.5 * (c->vertexy(k) + c->vertexy(k + 1)); c->celldy(k) = dy; }
  for (int k = -1; k <= ny + 2; ++k)
    for (int j = -1; j <= nx + 2; ++j) c->volume(j, k) = dx * dy;
  for (int k = -1; k <= ny + 2; ++k)
    for (int j = -1; j <= nx + 3; ++j) c->xarea(j, k) = c->celldy(k);
  for (int k = -1; k <= ny + 3; ++k)
    for (int j = -1; j <= nx + 2; ++j) c->yarea(j, k) = c->celldx(j);

  /* state edges nudged by dx/100 for rectangles (reading A6) */
  std::vector<oracle_state>& st = c->states;
  for (size_t n = 1; n < st.size(); ++n)
    if (st[n].geometry == OR_GEOM_RECT) {
      st[n].xmin = st[n].xmin + (dx / 100.0);
      st[n].ymin = st[n].ymin + (dy / 100.0);
      st[n].xmax = st[n].xmax - (dx / 100.0);
      st[n].ymax = st[n].ymax - (dy / 100.0);
    }

  /* generate_chunk: state 1 is the background */
  for (int k = -1; k <= ny + 2; ++k)
    for (int j = -1; j <= nx + 2; ++j) { c->energy0(j, k) = st[0].energy; c->density0(j, k) = st[0].density; }
  for (int k = -1; k <= ny + 3; ++k)
    for (int j = -1; j <= nx + 3; ++j) { c->xvel0(j, k) = st[0].xvel; c->yvel0(j, k) = st[0].yvel; }
  for (size_t s = 1; s < st.size(); ++s) {
    double x_cent = st[s].xmin, y_cent = st[s].ymin;
    for (int k = -1; k <= ny + 2; ++k)
      for (int j = -1; j <= nx + 2; ++j) {
        bool hit = false;
        if (st[s].geometry == OR_GEOM_RECT) {
          hit = c->vertexx(j + 1) >= st[s].xmin && c->vertexx(j) < st[s].xmax &&
                c->vertexy(k + 1) >= st[s].ymin && c->vertexy(k) < st[s].ymax;
        } else if (st[s].geometry == OR_GEOM_CIRCLE) {
          double radius = std::sqrt((c->cellx(j) - x_cent) * (c->cellx(j) - x_cent) +
                                    (c->celly(k) - y_cent) * (c->celly(k) - y_cent));
          hit = radius <= st[s].radius;
        } else if (st[s].geometry == OR_GEOM_POINT) {
          hit = c->vertexx(j) == x_cent && c->vertexy(k) == y_cent;
        }
        if (hit) {
          c->energy0(j, k) = st[s].energy;
          c->density0(j, k) = st[s].density;
          for (int kt = k; kt <= k + 1; ++kt)
            for (int jt = j; jt <= j + 1; ++jt) { c->xvel0(jt, kt) = st[s].xvel; c->yvel0(jt, kt) = st[s].yvel; }
        }
      }
  }
}

struct FieldDesc { Arr* a; int nxe, nye; FieldType t; };

FieldDesc field_desc(oracle_ctx* c, int fid) {
  const int nx = c->g.x_cells, ny = c->g.y_cells;
  switch (fid) {
    case OF_DENSITY0: return {&c->density0, nx, ny, CELL};
    case OF_ENERGY0: return {&c->energy0, nx, ny, CELL};
    case OF_PRESSURE: return {&c->pressure, nx, ny, CELL};
    case OF_VISCOSITY: return {&c->viscosity, nx, ny, CELL};
    case OF_SOUNDSPEED: return {&c->soundspeed, nx, ny, CELL};
    case OF_XVEL0: return {&c->xvel0, nx + 1, ny + 1, XVEL};
    case OF_YVEL0: return {&c->yvel0, nx + 1, ny + 1, YVEL};
    case OF_DENSITY1: return {&c->density1, nx, ny, CELL};
    case OF_ENERGY1: return {&c->energy1, nx, ny, CELL};
    case OF_XVEL1: return {&c->xvel1, nx + 1, ny + 1, XVEL};
    case OF_YVEL1: return {&c->yvel1, nx + 1, ny + 1, YVEL};
    case OF_VOL_FLUX_X: return {&c->vol_flux_x, nx + 1, ny, XFACE};
    case OF_VOL_FLUX_Y: return {&c->vol_flux_y, nx, ny + 1, YFACE};
    case OF_MASS_FLUX_X: return {&c->mass_flux_x, nx + 1, ny, XFACE};
    case OF_MASS_FLUX_Y: return {&c->mass_flux_y, nx, ny + 1, YFACE};
  }
  return {nullptr, 0, 0, CELL};
}

}  // namespace

extern "C" {

oracle_ctx* oracle_create(const oracle_grid* g, const oracle_state* s, int32_t nstates) {
  if (!g || !s || nstates < 1 || g->x_cells < 2 || g->y_cells < 2 || !(g->xmax > g->xmin) ||
      !(g->ymax > g->ymin))
    return nullptr;
  oracle_ctx* c = new oracle_ctx();
  c->g = *g;
  if (c->g.dtinit == 0.0) c->g.dtinit = 0.1;
  if (c->g.dtmax == 0.0) c->g.dtmax = 1.0;
  if (c->g.dtmin == 0.0) c->g.dtmin = 1.0e-7;
  if (c->g.dtrise == 0.0) c->g.dtrise = 1.5;
  if (c->g.dtc_safe == 0.0) c->g.dtc_safe = 0.7;
  if (c->g.dtu_safe == 0.0) c->g.dtu_safe = 0.5;
  if (c->g.dtv_safe == 0.0) c->g.dtv_safe = 0.5;
  if (c->g.dtdiv_safe == 0.0) c->g.dtdiv_safe = 0.7;
  c->states.assign(s, s + nstates);
  initialise(c);
  oracle_refresh(c);
  c->step = 0; c->time = 0.0; c->dtold = c->g.dtinit; c->dt = c->g.dtinit;
  c->advect_x = c->g.advect_x_first != 0;
  return c;
}

void oracle_refresh(oracle_ctx* c) {
  ideal_gas(c, false);
  reflect(c, c->density0, CELL, 2);
  reflect(c, c->energy0, CELL, 2);
  reflect(c, c->pressure, CELL, 2);
  reflect(c, c->viscosity, CELL, 2);
  reflect(c, c->density1, CELL, 2);
  reflect(c, c->energy1, CELL, 2);
  reflect(c, c->xvel0, XVEL, 2);
  reflect(c, c->yvel0, YVEL, 2);
  reflect(c, c->xvel1, XVEL, 2);
  reflect(c, c->yvel1, YVEL, 2);
}

void oracle_destroy(oracle_ctx* c) { delete c; }

int32_t oracle_step(oracle_ctx* c, int32_t n, double* dt_hist) {
  for (int i = 0; i < n; ++i) {
    int rc = full_step(c);
    if (rc) return rc;
    if (dt_hist) dt_hist[i] = c->dt;
  }
  return 0;
}

int32_t oracle_run_stage(oracle_ctx* c, int32_t stage) {
  switch (stage) {
    case OS_TIMESTEP: return timestep(c);
    case OS_PDV_PREDICT: pdv_predict_stage(c); return 0;
    case OS_ACCELERATE: accelerate(c); return 0;
    case OS_PDV_CORRECT: pdv(c, false); return 0;
    case OS_FLUX_CALC: flux_calc(c); return 0;
    case OS_ADVECTION: advection(c); return 0;
    case OS_RESET: finish_step(c); return 0;
    case OS_ADV_CELL1: advection_part(c, 0); return 0;
    case OS_ADV_MOM1: advection_part(c, 1); return 0;
    case OS_ADV_CELL2: advection_part(c, 2); return 0;
    case OS_ADV_MOM2: advection_part(c, 3); return 0;
  }
  return -1;
}

/* c.12 field_summary; compensated = 0: sequential accumulation in the
 * reference's loop order; 1: Neumaier compensated sums of the same terms. */
static void field_summary_impl(oracle_ctx* c, double* out, int compensated) {
  ideal_gas(c, false);
  double acc[5] = {0.0, 0.0, 0.0, 0.0, 0.0}, comp[5] = {0.0, 0.0, 0.0, 0.0, 0.0};
  for (int k = c->y_min; k <= c->y_max; ++k)
    for (int j = c->x_min; j <= c->x_max; ++j) {
      double vsqrd = 0.0;
      for (int kv = k; kv <= k + 1; ++kv)
        for (int jv = j; jv <= j + 1; ++jv)
          vsqrd = vsqrd + 0.25 * (c->xvel0(jv, kv) * c->xvel0(jv, kv) + c->yvel0(jv, kv) * c->yvel0(jv, kv));
      double cell_vol = c->volume(j, k);
      double cell_mass = cell_vol * c->density0(j, k);
      double term[5] = {cell_vol, cell_mass, cell_mass * c->energy0(j, k), cell_mass * 0.5 * vsqrd,
                        cell_vol * c->pressure(j, k)};
      for (int q = 0; q < 5; ++q) {
        if (!compensated) {
          acc[q] = acc[q] + term[q];
        } else {
          double t = acc[q] + term[q];
          if (std::fabs(acc[q]) >= std::fabs(term[q]))
            comp[q] += (acc[q] - t) + term[q];
          else
            comp[q] += (term[q] - t) + acc[q];
          acc[q] = t;
        }
      }
    }
  for (int q = 0; q < 5; ++q) out[q] = acc[q] + comp[q];
}

void oracle_field_summary(oracle_ctx* c, double* out) { field_summary_impl(c, out, 0); }

void oracle_field_summary_compensated(oracle_ctx* c, double* out) { field_summary_impl(c, out, 1); }

void oracle_clock(oracle_ctx* c, int32_t* step, double* time, double* dt, double* dtold) {
  if (step) *step = c->step;
  if (time) *time = c->time;
  if (dt) *dt = c->dt;
  if (dtold) *dtold = c->dtold;
}

int32_t oracle_read_field(oracle_ctx* c, int32_t fid, double* out, int64_t n) {
  FieldDesc d = field_desc(c, fid);
  if (!d.a || n != (int64_t)d.nxe * d.nye) return -1;
  for (int k = 1; k <= d.nye; ++k)
    for (int j = 1; j <= d.nxe; ++j) out[(size_t)(k - 1) * d.nxe + (j - 1)] = (*d.a)(j, k);
  return 0;
}

int32_t oracle_write_field(oracle_ctx* c, int32_t fid, const double* in, int64_t n) {
  FieldDesc d = field_desc(c, fid);
  if (!d.a || n != (int64_t)d.nxe * d.nye) return -1;
  for (int k = 1; k <= d.nye; ++k)
    for (int j = 1; j <= d.nxe; ++j) (*d.a)(j, k) = in[(size_t)(k - 1) * d.nxe + (j - 1)];
  return 0;
}

}  // extern "C"
