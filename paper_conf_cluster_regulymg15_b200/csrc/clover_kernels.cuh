// clover_kernels.cuh -- per-point arithmetic of one CloverLeaf 2D timestep.
//
// Method: sec. V (CloverLeaf 2D, compressible Euler, finite
// volume, staggered grid); per-kernel arithmetic as read in SURVEY.md 8(c)
// c.2-c.12, written here independently of the oracle.  Every expression keeps
// the reading's evaluation order, the library is compiled with -fmad=false
// and every division is correctly rounded (DivFast/DivIEEE, clover_common.cuh),
// so results are bitwise reproducible against any IEEE fp64 implementation
// of the same reading (reading A8).
//
// This file holds the per-point arithmetic of every step phase and the
// one-thread k_dt_finalize; the kernels that map it onto the mesh are in
// clover_stream.cuh.  Halo updates (a2, a4, a11, a13,
// a16) are folded into the producers' epilogues at reflective walls
// (store_field) and into copy/NCCL phases at chunk boundaries; reset_field
// (a18) is a buffer rotation.
//
// Per-point arithmetic lives in templated device functions taking the
// division policy; kernels run DivFast and redo a point with DivIEEE only
// when its sticky flag is set (tiny numerators, see clover_common.cuh).
#pragma once
#include "clover_common.cuh"

namespace clover {

// ---------------------------------------------------------------- c.2 EOS
__device__ __forceinline__ double eos_pressure(double rho, double e) {
  const double gm1 = 1.4 - 1.0;  // reading A2
  return gm1 * rho * e;
}

template <class D>
__device__ __forceinline__ double eos_soundspeed(D& dv, double rho, double e) {
  const double gm1 = 1.4 - 1.0;
  double v = dv.nz(1.0, rho);
  double p = gm1 * rho * e;
  double pbe = gm1 * rho;
  double pbv = -rho * p;
  double c2 = v * v * (p * pbe - pbv);
  return sqrt(c2);
}

// the square of the ideal_gas sound speed (eos_soundspeed = sqrt of this)
template <class D>
__device__ __forceinline__ double eos_c2(D& dv, double rho, double e) {
  const double gm1 = 1.4 - 1.0;
  double v = dv.nz(1.0, rho);
  double p = gm1 * rho * e;
  double pbe = gm1 * rho;
  double pbv = -rho * p;
  return v * v * (p * pbe - pbv);
}

__device__ __forceinline__ double eos_soundspeed_ieee(double rho, double e) {
  DivIEEE d;
  return eos_soundspeed(d, rho, e);
}

struct DtParams {
  double dtc_safe, dtu_safe, dtv_safe, dtdiv_safe;
  double dtrise, dtmax, dtmin;
};

// ------------------------------------------------ viscosity + calc_dt
struct ViscIn {
  double rho, e, pl, pr, pb, pt;
  double u00, u10, u01, u11, v00, v10, v01, v11;
};

// c.3 viscosity of one cell (writes q) and the square of the c.4 sound-speed
// term, cc2 = cs*cs + 2q/rho; the reading takes cc = max(sqrt(cc2), g_small)
// per cell, which only enters calc_dt through its maximum (DtAcc).
template <class D>
__device__ __forceinline__ void visc_cell(D& dv, const ViscIn& I, const Chunk& C, double& qv,
                                          double& cc2, double& c2) {
  const double dx = C.dx, dy = C.dy;
  const double u00 = I.u00, u10 = I.u10, u01 = I.u01, u11 = I.u11;
  const double v00 = I.v00, v10 = I.v10, v01 = I.v01, v11 = I.v11;
  double ugrad = (u10 + u11) - (u00 + u01);
  double vgrad = (v01 + v11) - (v00 + v10);
  double div = (dx * (ugrad) + dy * (vgrad));
  // The reading sets q = 0 when limiter > 0 or div >= 0; the limiter (and
  // the pressure gradients it needs) is only evaluated when div >= 0 does not
  // already decide it (same results; no work in non-compressing cells).
  qv = 0.0;
  if (!(div >= 0.0)) {
    double strain2 = dv.c(0.5 * (u01 + u11 - u00 - u10), dy, C.rdy) + dv.c(0.5 * (v10 + v11 - v00 - v01), dx, C.rdx);
    double pgradx = dv.c(I.pr - I.pl, dx + dx, C.r2dx);
    double pgrady = dv.c(I.pt - I.pb, dy + dy, C.r2dy);
    double pgradx2 = pgradx * pgradx;
    double pgrady2 = pgrady * pgrady;
    double limiter = dv(dv.c(0.5 * (ugrad), dx, C.rdx) * pgradx2 + dv.c(0.5 * (vgrad), dy, C.rdy) * pgrady2 +
                            strain2 * pgradx * pgrady,
                        fmax(pgradx2 + pgrady2, 1.0e-16));
    if (!(limiter > 0.0)) {
      pgradx = copysign(fmax(1.0e-16, fabs(pgradx)), pgradx);
      pgrady = copysign(fmax(1.0e-16, fabs(pgrady)), pgrady);
      double pgrad = sqrt(pgradx * pgradx + pgrady * pgrady);
      double xgrad = fabs(dv(dx * pgrad, pgradx));
      double ygrad = fabs(dv(dy * pgrad, pgrady));
      double grad = fmin(xgrad, ygrad);
      double grad2 = grad * grad;
      qv = 2.0 * I.rho * grad2 * limiter * limiter;
    }
  }
  // c2 = cs^2 before the square root (ideal_gas).  Where q = 0 the reading's
  // cc2 = RN(RN(sqrt(c2))^2) + RN(2q/rho) is f(c2) = RN(RN(sqrt(c2))^2), a
  // monotone function of c2, so DtAcc keeps max c2 over those cells and
  // applies f once; cells with q != 0 evaluate cc2 here.
  c2 = eos_c2(dv, I.rho, I.e);
  cc2 = 0.0;
  if (qv != 0.0) {
    const double cs = sqrt(c2);
    cc2 = cs * cs + dv(2.0 * qv, I.rho);
  }
}

// c.4 calc_dt, reduced over a set of cells without per-cell divisions.
// Per cell the reading takes
//   dt_cell = min( A_c / cc, A_u / du, A_v / dv', dtdiv_safe * (-1 / (w / 2vol)) )
// (the last term only when w / 2vol < -g_small, else g_big), with A_c, A_u,
// A_v and 2vol launch constants and every quotient correctly rounded.
// Correct rounding is monotone (x <= y => RN(x) <= RN(y)), so the minimum
// over cells of RN(A / d) is RN(A / max d), that of RN(w / 2vol) is
// RN(min w / 2vol), and -1/x grows with x < 0: the minimum of the per-cell
// dt over the set equals the dt computed once from the four extremes below,
// bit for bit.  The kernel keeps the extremes per thread and divides once.
// Likewise correctly rounded sqrt and fmax(., g_small) are monotone, so the
// maximum over cells of cc = fmax(sqrt(cc2), g_small) is fmax(sqrt(max cc2),
// g_small): one square root per thread instead of one per cell.
//
// Faces: |dv1| / |dv2| of a cell are the magnitudes of its left/right (u) and
// bottom/top (v) face volume terms; the left face of cell j is bitwise the
// right face of cell j-1 (same expression of the same node velocities), and
// the bottom face of row k the top face of row k-1.  The maximum over a set
// of cells is therefore the maximum over the set's faces, each taken once:
// add() takes the right and top faces of every cell, plus the left face
// when the caller's column has no left neighbour in the reduction (chunk
// column 1); the bottom face of a segment's first row comes from bottom().
// The g_small*vol floor of every per-cell term is applied once in dt()
// (max is associative).  Non-negative, non-NaN operands: the compare-select
// max equals fmax bit for bit.
__device__ __forceinline__ double dmax_nn(double a, double b) { return b > a ? b : a; }

struct DtAcc {
  double c2max = 0.0, ccqmax = 0.0, dumax = 0.0, dvmax = 0.0, wmin = G_BIG;
  __device__ __forceinline__ void add(const ViscIn& I, const Chunk& C, double qv, double cc2,
                                      double c2, bool left) {
    const double dx = C.dx, dy = C.dy;
    double dvv = 0.0;
    double dv1 = (I.u00 + I.u01) * dy;
    double dv2 = (I.u10 + I.u11) * dy;
    dvv = dvv + dv2 - dv1;
    dumax = dmax_nn(dumax, fabs(dv2));
    if (left) dumax = dmax_nn(dumax, fabs(dv1));
    dv1 = (I.v00 + I.v10) * dx;
    dv2 = (I.v01 + I.v11) * dx;
    dvv = dvv + dv2 - dv1;
    dvmax = dmax_nn(dvmax, fabs(dv2));
    wmin = dvv < wmin ? dvv : wmin;
    if (qv != 0.0) ccqmax = dmax_nn(ccqmax, cc2);
    else c2max = dmax_nn(c2max, c2);
  }
  // bottom face of the first row: v at nodes (j, k0) and (j+1, k0)
  __device__ __forceinline__ void bottom(double v00, double v10, const Chunk& C) {
    dvmax = dmax_nn(dvmax, fabs((v00 + v10) * C.dx));
  }
  // dt of the set (call only if at least one cell was added)
  __device__ __forceinline__ double dt(const Chunk& C, const DtParams& prm) const {
    const double dx = C.dx, dy = C.dy, vol = dx * dy;
    const double cs = sqrt(c2max);
    const double ccmax = fmax(sqrt(dmax_nn(cs * cs, ccqmax)), G_SMALL);
    const double dum = fmax(dumax, G_SMALL * vol), dvm = fmax(dvmax, G_SMALL * vol);
    double dtct = div_fast_nz(prm.dtc_safe * fmin(dx, dy), ccmax);
    double dtut = div_fast_nz(prm.dtu_safe * 2.0 * vol, dum);
    double dtvt = div_fast_nz(prm.dtv_safe * 2.0 * vol, dvm);
    double dvv = wmin / (2.0 * vol);
    double dtdivt = (dvv < -G_SMALL) ? prm.dtdiv_safe * div_fast_nz(-1.0, dvv) : G_BIG;
    return fmin(fmin(dtct, dtut), fmin(dtvt, dtdivt));
  }
};

// ------------------------------------------------ k_dt_finalize (c.4 tail)
// dt = min(cells, dtold*dtrise, dtmax), small-dt check, clock, history and
// slot reset: one thread, after every contribution to dt_slot is visible.
__device__ __forceinline__ void dt_finalize(StepScalars* __restrict__ s, double* __restrict__ hist,
                                            const DtParams& prm) {
  double dtc = __longlong_as_double((long long)*(volatile unsigned long long*)&s->dt_slot);
  double dt = fmin(fmin(dtc, (s->dtold * prm.dtrise)), prm.dtmax);
  s->dt = dt;
  if (dt < prm.dtmin) {
    if (s->err == 0) s->err = -5;  // CLOVER_ERR_SMALL_DT
  } else {
    s->dtold = dt;
  }
  s->time = s->time + dt;
  s->step = s->step + 1;
  hist[(s->step - 1) % DT_HIST] = dt;
  s->dt_slot = (unsigned long long)__double_as_longlong(G_BIG);
}

// separate launch: multi-chunk / multi-rank steps (after the NCCL MIN)
__global__ void k_dt_finalize(StepScalars* __restrict__ s, double* __restrict__ hist,
                              DtParams prm) {
  pdl_trigger();
  pdl_wait();
  dt_finalize(s, hist, prm);
}

// ------------------------------------------------ Lagrangian phase (c.5-c.7)
// PdV predictor (predict=T) + ideal_gas(predict): half-step pressure of one
// cell from its 4 node velocities (a,b = left face nodes bottom/top;
// c,d = right face; va,vb = bottom face nodes left/right; vc,vd = top face).
// The y-face flux terms of the predictor: the top face of row k is the
// bottom face of row k+1, the same expression of the same two node
// velocities, so the row-streaming kernel carries it (pdv_face_pred).
__device__ __forceinline__ double pdv_face_pred(double a, double b, double d, double dt) {
  return (d * (a + b + a + b)) * 0.25 * dt * 0.5;
}
template <class D>
__device__ __forceinline__ double pdv_predict_pressure_bt(D& dv, double r, double e, double q,
                                                          double ua, double ub, double uc,
                                                          double ud, double bottom_flux,
                                                          double top_flux, double dx, double dy,
                                                          double rvol, double dt) {
  const double vol = dx * dy;
  double left_flux = pdv_face_pred(ua, ub, dy, dt);
  double right_flux = pdv_face_pred(uc, ud, dy, dt);
  double total_flux = right_flux - left_flux + top_flux - bottom_flux;
  double volume_change = dv.nz(vol, vol + total_flux);
  double recip_volume = rvol;  // = RN(1.0/vol), precomputed
  double p0 = eos_pressure(r, e);
  double energy_change = (dv(p0, r) + dv(q, r)) * total_flux * recip_volume;
  double e1p = e - energy_change;
  double d1p = r * volume_change;
  return eos_pressure(d1p, e1p);
}
template <class D>
__device__ __forceinline__ double pdv_predict_pressure(D& dv, double r, double e, double q,
                                                       double ua, double ub, double uc, double ud,
                                                       double va, double vb, double vc, double vd,
                                                       double dx, double dy, double rvol, double dt) {
  return pdv_predict_pressure_bt(dv, r, e, q, ua, ub, uc, ud, pdv_face_pred(va, vb, dx, dt),
                                 pdv_face_pred(vc, vd, dx, dt), dx, dy, rvol, dt);
}

// accelerate (c.6) at one node: cells ordered (j-1,k-1), (j,k-1), (j,k), (j-1,k).
// mm[i] = rr[i] * vol: the cell masses; the row-streaming kernel carries the
// two of row k-1 from the previous node row (same products, same bits).
template <class D>
__device__ __forceinline__ void accelerate_node_m(D& dv, const double* mm, const double* pp,
                                                  const double* qq, double u0v, double v0v,
                                                  double dx, double dy, double dt, double& uu,
                                                  double& vv) {
  const double halfdt = 0.5 * dt;
  double nodal_mass = (mm[0] + mm[1] + mm[2] + mm[3]) * 0.25;
  double stepbymass = dv.nz(halfdt, nodal_mass);
  uu = u0v - stepbymass * (dy * (pp[2] - pp[3]) + dy * (pp[1] - pp[0]));
  vv = v0v - stepbymass * (dx * (pp[2] - pp[1]) + dx * (pp[3] - pp[0]));
  uu = uu - stepbymass * (dy * (qq[2] - qq[3]) + dy * (qq[1] - qq[0]));
  vv = vv - stepbymass * (dx * (qq[2] - qq[1]) + dx * (qq[3] - qq[0]));
}

template <class D>
__device__ __forceinline__ void accelerate_node(D& dv, const double* rr, const double* pp,
                                                const double* qq, double u0v, double v0v,
                                                double dx, double dy, double dt, double& uu,
                                                double& vv) {
  const double vol = dx * dy;
  const double halfdt = 0.5 * dt;
  double nodal_mass = (rr[0] * vol + rr[1] * vol + rr[2] * vol + rr[3] * vol) * 0.25;
  double stepbymass = dv.nz(halfdt, nodal_mass);
  // p(j,k)=pp[2], p(j-1,k)=pp[3], p(j,k-1)=pp[1], p(j-1,k-1)=pp[0]
  uu = u0v - stepbymass * (dy * (pp[2] - pp[3]) + dy * (pp[1] - pp[0]));
  vv = v0v - stepbymass * (dx * (pp[2] - pp[1]) + dx * (pp[3] - pp[0]));
  uu = uu - stepbymass * (dy * (qq[2] - qq[3]) + dy * (qq[1] - qq[0]));
  vv = vv - stepbymass * (dx * (qq[2] - qq[1]) + dx * (qq[3] - qq[0]));
}

// PdV corrector (predict=F) for one cell; returns energy1, density1.
// corrector face flux from a face's summed velocities (the top face of row
// k is the bottom face of row k+1: carried by the kernel)
__device__ __forceinline__ double pdv_face_corr(double sum, double d, double dt) {
  return (d * sum) * 0.25 * dt;
}
template <class D>
__device__ __forceinline__ void pdv_correct_bt(D& dv, double r, double e, double ph, double q,
                                               double lsum, double rsum, double bottom_flux,
                                               double top_flux, double dx, double dy, double rvol,
                                               double dt, double& e1v, double& d1v) {
  const double vol = dx * dy;
  double left_flux = pdv_face_corr(lsum, dy, dt);
  double right_flux = pdv_face_corr(rsum, dy, dt);
  double total_flux = right_flux - left_flux + top_flux - bottom_flux;
  const double new_vol = vol + total_flux;
  double volume_change = dv.nz(vol, new_vol);
  dv.vol_check(new_vol);  // CLOVER_ERR_NEG_VOLUME (kf_lagrangian latches it)
  double recip_volume = rvol;  // = RN(1.0/vol), precomputed
  double energy_change = (dv(ph, r) + dv(q, r)) * total_flux * recip_volume;
  e1v = e - energy_change;
  d1v = r * volume_change;
}
template <class D>
__device__ __forceinline__ void pdv_correct(D& dv, double r, double e, double ph, double q,
                                            double lsum, double rsum, double bsum, double tsum,
                                            double dx, double dy, double rvol, double dt, double& e1v,
                                            double& d1v) {
  pdv_correct_bt(dv, r, e, ph, q, lsum, rsum, pdv_face_corr(bsum, dx, dt),
                 pdv_face_corr(tsum, dx, dt), dx, dy, rvol, dt, e1v, d1v);
}

// ------------------------------------------------ advec_cell (c.8)
// a / b for b > 0: a zero numerator (the common case in quiescent regions)
// is its own quotient (+0/b = +0, -0/b = -0), so the division may be
// skipped.  Off by default: measured at 3840^2 the per-division branch
// saves 0.018 ms/step on the bm deck but costs 0.10 ms/step on a fully
// active flow (compare + branch per division, bench.py active_flow).
#ifndef CLOVER_DIV_SKIP
#define CLOVER_DIV_SKIP 0
#endif
template <class D>
__device__ __forceinline__ double div_pos(D& dv, double a, double b) {
#if CLOVER_DIV_SKIP
  double q = a;
  if (a != 0.0) q = dv(a, b);
  return q;
#else
  return dv(a, b);
#endif
}
constexpr double ONE_BY_SIX = 1.0 / 6.0;

// Donor-cell flux with the limiter of c.8 for one face.  pv_don = pre_vol of
// the donor cell; r*/e* = density/energy at upwind, donor, downwind.
template <class D>
__device__ __forceinline__ void cell_face_flux(D& dv, double F, double pv_don, double ru, double rd,
                                               double rw, double eu, double ed, double ew,
                                               double& mflux, double& eflux) {
  double sigmat = div_pos(dv, fabs(F), pv_don);
  double sigma3 = (1.0 + sigmat);  // * (vertexdx(j)/vertexdx(dif)) == 1 exactly (uniform mesh)
  double sigma4 = 2.0 - sigmat;
  double diffuw = rd - ru;
  double diffdw = rw - rd;
  double wind = 1.0;
  if (diffdw <= 0.0) wind = -1.0;
  double limiter;
  if (diffuw * diffdw > 0.0)
    limiter = (1.0 - sigmat) * wind *
              fmin(fmin(fabs(diffuw), fabs(diffdw)),
                   ONE_BY_SIX * (sigma3 * fabs(diffuw) + sigma4 * fabs(diffdw)));
  else
    limiter = 0.0;
  mflux = F * (rd + limiter);
  double sigmam = div_pos(dv, fabs(mflux), rd * pv_don);
  diffuw = ed - eu;
  diffdw = ew - ed;
  wind = 1.0;
  if (diffdw <= 0.0) wind = -1.0;
  if (diffuw * diffdw > 0.0)
    limiter = (1.0 - sigmam) * wind *
              fmin(fmin(fabs(diffuw), fabs(diffdw)),
                   ONE_BY_SIX * (sigma3 * fabs(diffuw) + sigma4 * fabs(diffdw)));
  else
    limiter = 0.0;
  eflux = mflux * (ed + limiter);
}

// advec_cell cell update: returns density and energy after the sweep.
template <class D>
__device__ __forceinline__ void cell_update(D& dv, double rho, double en, double pv, double mlo,
                                            double mhi, double eflo, double efhi, double flo,
                                            double fhi, double& rout, double& eout) {
  double pre_mass = rho * pv;
  double post_mass = pre_mass + mlo - mhi;
  double post_ener = dv(en * pre_mass + eflo - efhi, post_mass);
  double advec_vol = pv + flo - fhi;
  rout = dv(post_mass, advec_vol);
  eout = post_ener;
}

// ------------------------------------------------ advec_mom (c.9)
// Momentum flux at one node for one velocity component (limited, c.9),
// given sigma = |node_flux| / node_mass_pre(donor).
template <class D>
__device__ __forceinline__ double mom_flux(D& dv, double nf, double sigma, double vup,
                                           double vdon, double vdw, double width, double rwidth) {
  // width = celldx(j) and celldx(dif) are the same constant on the uniform mesh
  double vdiffuw = vdon - vup;
  double vdiffdw = vdw - vdon;
  double limiter = 0.0;
  if (vdiffuw * vdiffdw > 0.0) {
    double auw = fabs(vdiffuw);
    double adw = fabs(vdiffdw);
    double wind = 1.0;
    if (vdiffdw <= 0.0) wind = -1.0;
    limiter = wind * fmin(fmin(dv.c(width * (dv.c((2.0 - sigma) * adw, width, rwidth) +
                                             dv.c((1.0 + sigma) * auw, width, rwidth)),
                                    6.0, ONE_BY_SIX),
                               auw), adw);
  }
  double advec_vel = vdon + (1.0 - sigma) * limiter;
  return advec_vel * nf;
}

// both velocity components at one node: the reference evaluates sigma in
// each component's loop from the same node flux and mass, so one division
// serves both (same bits)
template <class D>
__device__ __forceinline__ void mom_flux2(D& dv, double nf, double nmp, const double* uu,
                                          const double* vv, double w, double rw, double& mu,
                                          double& mv) {
  const double sigma = div_pos(dv, fabs(nf), nmp);
  mu = mom_flux(dv, nf, sigma, uu[0], uu[1], uu[2], w, rw);
  mv = mom_flux(dv, nf, sigma, vv[0], vv[1], vv[2], w, rw);
}

template <class D>
__device__ __forceinline__ void mom_update(D& dv, double u, double v, double pre, double post,
                                           double mulo, double muhi, double mvlo, double mvhi,
                                           double& un, double& vn) {
  un = div_pos(dv, u * pre + mulo - muhi, post);
  vn = div_pos(dv, v * pre + mvlo - mvhi, post);
}

}  // namespace clover
