// clover_kernels.cuh -- sm_100a kernels of one CloverLeaf 2D timestep.
//
// Method: sec. V (CloverLeaf 2D, compressible Euler, finite
// volume, staggered grid); per-kernel arithmetic as read in SURVEY.md 8(c)
// c.2-c.12, written here independently of the oracle.  Every expression keeps
// the reading's evaluation order, the library is compiled with -fmad=false
// and every division is correctly rounded (DivFast/DivIEEE, clover_common.cuh),
// so results are bitwise reproducible against any IEEE fp64 implementation
// of the same reading (reading A8).
//
// Kernel groups per step:
//   k_visc_dt      ideal_gas + viscosity + calc_dt + block min   (a1-a5)
//   k_dt_finalize  dt = min(cells, dtold*dtrise, dtmax), clock   (a5)
//   k_lagrangian   PdV predictor + ideal_gas + accelerate +
//                  PdV corrector + flux_calc, ring-recompute tile (a6-a10)
//   k_advec_cell_{x,y}   advec_cell sweep                         (a12/a15)
//   k_advec_mom_{x,y}    advec_mom sweep for u and v together     (a14/a17)
// Halo updates (a2, a4, a11, a13, a16) are folded into the producers'
// epilogues at reflective walls (store_field) and into copy/NCCL phases at
// chunk boundaries; reset_field (a18) is a buffer rotation.
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
  double v = dv(1.0, rho);
  double p = gm1 * rho * e;
  double pbe = gm1 * rho;
  double pbv = -rho * p;
  double c2 = v * v * (p * pbe - pbv);
  return sqrt(c2);
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

// c.3 viscosity then c.4 calc_dt for one cell; returns dt_cell, writes q.
template <class D>
__device__ __forceinline__ double visc_dt_cell(D& dv, const ViscIn& I, double dx, double dy,
                                               const DtParams& prm, double& qv) {
  const double u00 = I.u00, u10 = I.u10, u01 = I.u01, u11 = I.u11;
  const double v00 = I.v00, v10 = I.v10, v01 = I.v01, v11 = I.v11;
  double ugrad = (u10 + u11) - (u00 + u01);
  double vgrad = (v01 + v11) - (v00 + v10);
  double div = (dx * (ugrad) + dy * (vgrad));
  double strain2 = dv(0.5 * (u01 + u11 - u00 - u10), dy) + dv(0.5 * (v10 + v11 - v00 - v01), dx);
  double pgradx = dv(I.pr - I.pl, dx + dx);
  double pgrady = dv(I.pt - I.pb, dy + dy);
  double pgradx2 = pgradx * pgradx;
  double pgrady2 = pgrady * pgrady;
  double limiter = dv(dv(0.5 * (ugrad), dx) * pgradx2 + dv(0.5 * (vgrad), dy) * pgrady2 +
                          strain2 * pgradx * pgrady,
                      fmax(pgradx2 + pgrady2, 1.0e-16));
  if ((limiter > 0.0) || (div >= 0.0)) {
    qv = 0.0;
  } else {
    pgradx = copysign(fmax(1.0e-16, fabs(pgradx)), pgradx);
    pgrady = copysign(fmax(1.0e-16, fabs(pgrady)), pgrady);
    double pgrad = sqrt(pgradx * pgradx + pgrady * pgrady);
    double xgrad = fabs(dv(dx * pgrad, pgradx));
    double ygrad = fabs(dv(dy * pgrad, pgrady));
    double grad = fmin(xgrad, ygrad);
    double grad2 = grad * grad;
    qv = 2.0 * I.rho * grad2 * limiter * limiter;
  }
  const double vol = dx * dy;
  double cs = eos_soundspeed(dv, I.rho, I.e);
  double cc = cs * cs;
  cc = cc + dv(2.0 * qv, I.rho);
  cc = fmax(sqrt(cc), G_SMALL);
  double dtct = dv(prm.dtc_safe * fmin(dx, dy), cc);
  double dvv = 0.0;
  double dv1 = (u00 + u01) * dy;
  double dv2 = (u10 + u11) * dy;
  dvv = dvv + dv2 - dv1;
  double dtut = dv(prm.dtu_safe * 2.0 * vol, fmax(fmax(fabs(dv1), fabs(dv2)), G_SMALL * vol));
  dv1 = (v00 + v10) * dx;
  dv2 = (v01 + v11) * dx;
  dvv = dvv + dv2 - dv1;
  double dtvt = dv(prm.dtv_safe * 2.0 * vol, fmax(fmax(fabs(dv1), fabs(dv2)), G_SMALL * vol));
  dvv = dv(dvv, 2.0 * vol);
  double dtdivt = (dvv < -G_SMALL) ? prm.dtdiv_safe * dv(-1.0, dvv) : G_BIG;
  return fmin(fmin(dtct, dtut), fmin(dtvt, dtdivt));
}

// ------------------------------------------------ k_visc_dt  (c.2, c.3, c.4)
// One thread per interior cell.  Pressure at the 5-point stencil is
// recomputed from density0/energy0 (their halos are valid), so the stored
// pressure field of the reference is never materialised.
__global__ void __launch_bounds__(256)
k_visc_dt(Chunk c, const double* __restrict__ d0, const double* __restrict__ e0,
          const double* __restrict__ u0, const double* __restrict__ v0, double* __restrict__ q,
          StepScalars* __restrict__ s, DtParams prm) {
  const int j = blockIdx.x * blockDim.x + threadIdx.x + 1;
  const int k = blockIdx.y * blockDim.y + threadIdx.y + 1;
  double dtl = G_BIG;
  if (j <= c.nx && k <= c.ny) {
    const int i = idx(c, j, k);
    const int P = c.pitch;
    ViscIn I;
    I.rho = d0[i];
    I.e = e0[i];
    I.pl = eos_pressure(d0[i - 1], e0[i - 1]);
    I.pr = eos_pressure(d0[i + 1], e0[i + 1]);
    I.pb = eos_pressure(d0[i - P], e0[i - P]);
    I.pt = eos_pressure(d0[i + P], e0[i + P]);
    I.u00 = u0[i]; I.u10 = u0[i + 1]; I.u01 = u0[i + P]; I.u11 = u0[i + P + 1];
    I.v00 = v0[i]; I.v10 = v0[i + 1]; I.v01 = v0[i + P]; I.v11 = v0[i + P + 1];
    double qv;
    DivFast f;
    dtl = visc_dt_cell(f, I, c.dx, c.dy, prm, qv);
    if (f.bad) {
      DivIEEE x;
      dtl = visc_dt_cell(x, I, c.dx, c.dy, prm, qv);
    }
    store_field(c, q, K_CELL, j, k, qv);
  }
  // exact min: warp shuffle, then one atomicMin per CTA on the bit pattern
  // (positive doubles order like their unsigned bit patterns).
  for (int o = 16; o > 0; o >>= 1) dtl = fmin(dtl, __shfl_xor_sync(0xffffffffu, dtl, o));
  __shared__ double wmin[32];
  const int lane = (threadIdx.y * blockDim.x + threadIdx.x) & 31;
  const int warp = (threadIdx.y * blockDim.x + threadIdx.x) >> 5;
  if (lane == 0) wmin[warp] = dtl;
  __syncthreads();
  if (warp == 0) {
    const int nw = (blockDim.x * blockDim.y + 31) >> 5;
    double m = lane < nw ? wmin[lane] : G_BIG;
    for (int o = 16; o > 0; o >>= 1) m = fmin(m, __shfl_xor_sync(0xffffffffu, m, o));
    if (lane == 0) atomicMin(&s->dt_slot, (unsigned long long)__double_as_longlong(m));
  }
}

// ------------------------------------------------ k_dt_finalize (c.4 tail)
__global__ void k_dt_finalize(StepScalars* __restrict__ s, double* __restrict__ hist,
                              DtParams prm) {
  double dtc = __longlong_as_double((long long)s->dt_slot);
  double dt = fmin(fmin(dtc, (s->dtold * prm.dtrise)), prm.dtmax);
  s->dt = dt;
  if (dt < prm.dtmin) {
    if (s->err == 0) s->err = -5;
  } else {
    s->dtold = dt;
  }
  s->time = s->time + dt;
  s->step = s->step + 1;
  hist[(s->step - 1) % DT_HIST] = dt;
  s->dt_slot = (unsigned long long)__double_as_longlong(G_BIG);
}

// ------------------------------------------------ Lagrangian phase (c.5-c.7)
// PdV predictor (predict=T) + ideal_gas(predict): half-step pressure of one
// cell from its 4 node velocities (a,b = left face nodes bottom/top;
// c,d = right face; va,vb = bottom face nodes left/right; vc,vd = top face).
template <class D>
__device__ __forceinline__ double pdv_predict_pressure(D& dv, double r, double e, double q,
                                                       double ua, double ub, double uc, double ud,
                                                       double va, double vb, double vc, double vd,
                                                       double dx, double dy, double dt) {
  const double vol = dx * dy;
  double left_flux = (dy * (ua + ub + ua + ub)) * 0.25 * dt * 0.5;
  double right_flux = (dy * (uc + ud + uc + ud)) * 0.25 * dt * 0.5;
  double bottom_flux = (dx * (va + vb + va + vb)) * 0.25 * dt * 0.5;
  double top_flux = (dx * (vc + vd + vc + vd)) * 0.25 * dt * 0.5;
  double total_flux = right_flux - left_flux + top_flux - bottom_flux;
  double volume_change = dv(vol, vol + total_flux);
  double recip_volume = dv(1.0, vol);
  double p0 = eos_pressure(r, e);
  double energy_change = (dv(p0, r) + dv(q, r)) * total_flux * recip_volume;
  double e1p = e - energy_change;
  double d1p = r * volume_change;
  return eos_pressure(d1p, e1p);
}

// accelerate (c.6) at one node: cells ordered (j-1,k-1), (j,k-1), (j,k), (j-1,k).
template <class D>
__device__ __forceinline__ void accelerate_node(D& dv, const double* rr, const double* pp,
                                                const double* qq, double u0v, double v0v,
                                                double dx, double dy, double dt, double& uu,
                                                double& vv) {
  const double vol = dx * dy;
  const double halfdt = 0.5 * dt;
  double nodal_mass = (rr[0] * vol + rr[1] * vol + rr[2] * vol + rr[3] * vol) * 0.25;
  double stepbymass = dv(halfdt, nodal_mass);
  // p(j,k)=pp[2], p(j-1,k)=pp[3], p(j,k-1)=pp[1], p(j-1,k-1)=pp[0]
  uu = u0v - stepbymass * (dy * (pp[2] - pp[3]) + dy * (pp[1] - pp[0]));
  vv = v0v - stepbymass * (dx * (pp[2] - pp[1]) + dx * (pp[3] - pp[0]));
  uu = uu - stepbymass * (dy * (qq[2] - qq[3]) + dy * (qq[1] - qq[0]));
  vv = vv - stepbymass * (dx * (qq[2] - qq[1]) + dx * (qq[3] - qq[0]));
}

// PdV corrector (predict=F) for one cell; returns energy1, density1.
template <class D>
__device__ __forceinline__ void pdv_correct(D& dv, double r, double e, double ph, double q,
                                            double lsum, double rsum, double bsum, double tsum,
                                            double dx, double dy, double dt, double& e1v,
                                            double& d1v) {
  const double vol = dx * dy;
  double left_flux = (dy * lsum) * 0.25 * dt;
  double right_flux = (dy * rsum) * 0.25 * dt;
  double bottom_flux = (dx * bsum) * 0.25 * dt;
  double top_flux = (dx * tsum) * 0.25 * dt;
  double total_flux = right_flux - left_flux + top_flux - bottom_flux;
  double volume_change = dv(vol, vol + total_flux);
  double recip_volume = dv(1.0, vol);
  double energy_change = (dv(ph, r) + dv(q, r)) * total_flux * recip_volume;
  e1v = e - energy_change;
  d1v = r * volume_change;
}

// ------------------------------------------------ k_lagrangian
// Tile of LX x LY cells per CTA.  The PdV predictor + EOS run on the tile
// plus a 1-cell ring (accelerate at the tile's nodes needs the half-step
// pressure of all 4 surrounding cells); at reflective walls the ring takes
// the mirror of the tile's own results, exactly like the reference's
// update_halo{pressure} after the predictor.
constexpr int LX = 32, LY = 8;

__global__ void __launch_bounds__(LX * LY)
k_lagrangian(Chunk c, const double* __restrict__ d0, const double* __restrict__ e0,
             const double* __restrict__ u0, const double* __restrict__ v0,
             const double* __restrict__ q, double* __restrict__ d1, double* __restrict__ e1,
             double* __restrict__ u1, double* __restrict__ v1, double* __restrict__ fx,
             double* __restrict__ fy, const StepScalars* __restrict__ s) {
  constexpr int CW = LX + 2, CH = LY + 2;  // cell ring  [J0-1, J0+LX] x [K0-1, K0+LY]
  constexpr int NW = LX + 3, NH = LY + 3;  // node ring  [J0-1, J0+LX+1] x [K0-1, K0+LY+1]
  constexpr int AW = LX + 1, AH = LY + 1;  // accel nodes [J0, J0+LX] x [K0, K0+LY]
  __shared__ double sR[CH][CW], sE[CH][CW], sQ[CH][CW], sPh[CH][CW];
  __shared__ double sU0[NH][NW], sV0[NH][NW];
  __shared__ double sU1[AH][AW], sV1[AH][AW];

  const int J0 = blockIdx.x * LX + 1, K0 = blockIdx.y * LY + 1;
  const int tid = threadIdx.y * LX + threadIdx.x;
  const double dt = s->dt;
  const double dx = c.dx, dy = c.dy;

  for (int t = tid; t < CW * CH; t += LX * LY) {
    const int jj = t % CW, kk = t / CW;
    const int j = J0 - 1 + jj, k = K0 - 1 + kk;
    double r = 1.0, e = 0.0, qq = 0.0;
    if (j <= c.nx + HALO && k <= c.ny + HALO) {
      const int i = idx(c, j, k);
      r = d0[i]; e = e0[i]; qq = q[i];
    }
    sR[kk][jj] = r; sE[kk][jj] = e; sQ[kk][jj] = qq;
  }
  for (int t = tid; t < NW * NH; t += LX * LY) {
    const int jj = t % NW, kk = t / NW;
    const int j = J0 - 1 + jj, k = K0 - 1 + kk;
    double uu = 0.0, vv = 0.0;
    if (j <= c.nx + 1 + HALO && k <= c.ny + 1 + HALO) {
      const int i = idx(c, j, k);
      uu = u0[i]; vv = v0[i];
    }
    sU0[kk][jj] = uu; sV0[kk][jj] = vv;
  }
  __syncthreads();

  // PdV predictor + ideal_gas(predict) on the ring cells that are interior
  // or lie across a chunk boundary.
  for (int t = tid; t < CW * CH; t += LX * LY) {
    const int jj = t % CW, kk = t / CW;
    const int j = J0 - 1 + jj, k = K0 - 1 + kk;
    const bool outside_x = (j < 1 && c.wl) || (j > c.nx && c.wr) || j > c.nx + 1;
    const bool outside_y = (k < 1 && c.wb) || (k > c.ny && c.wt) || k > c.ny + 1;
    double ph = 0.0;
    if (!outside_x && !outside_y) {
      const double ua = sU0[kk][jj], ub = sU0[kk + 1][jj];
      const double uc = sU0[kk][jj + 1], ud = sU0[kk + 1][jj + 1];
      const double va = sV0[kk][jj], vb = sV0[kk][jj + 1];
      const double vc = sV0[kk + 1][jj], vd = sV0[kk + 1][jj + 1];
      const double r = sR[kk][jj], e = sE[kk][jj], qq = sQ[kk][jj];
      DivFast f;
      ph = pdv_predict_pressure(f, r, e, qq, ua, ub, uc, ud, va, vb, vc, vd, dx, dy, dt);
      if (f.bad) {
        DivIEEE x;
        ph = pdv_predict_pressure(x, r, e, qq, ua, ub, uc, ud, va, vb, vc, vd, dx, dy, dt);
      }
    }
    sPh[kk][jj] = ph;
  }
  __syncthreads();
  // reflective walls: ring pressure = mirror of the interior result
  for (int t = tid; t < CW * CH; t += LX * LY) {
    const int jj = t % CW, kk = t / CW;
    const int j = J0 - 1 + jj, k = K0 - 1 + kk;
    int js = j, ks = k;
    if (c.wl && j < 1) js = 1 - j;
    if (c.wr && j > c.nx && j <= c.nx + 1) js = 2 * c.nx + 1 - j;
    if (c.wb && k < 1) ks = 1 - k;
    if (c.wt && k > c.ny && k <= c.ny + 1) ks = 2 * c.ny + 1 - k;
    if (js != j || ks != k) sPh[kk][jj] = sPh[ks - (K0 - 1)][js - (J0 - 1)];
  }
  __syncthreads();

  // accelerate on nodes [J0, J0+LX] x [K0, K0+LY]
  for (int t = tid; t < AW * AH; t += LX * LY) {
    const int jj = t % AW, kk = t / AW;
    const int j = J0 + jj, k = K0 + kk;
    double uu = 0.0, vv = 0.0;
    if (j <= c.nx + 1 && k <= c.ny + 1) {
      // cell (j,k) is ring entry (jj+1, kk+1); (j-1,k-1) is (jj, kk)
      const int cj = jj + 1, ck = kk + 1;
      const double rr[4] = {sR[ck - 1][cj - 1], sR[ck - 1][cj], sR[ck][cj], sR[ck][cj - 1]};
      const double pp[4] = {sPh[ck - 1][cj - 1], sPh[ck - 1][cj], sPh[ck][cj], sPh[ck][cj - 1]};
      const double qq[4] = {sQ[ck - 1][cj - 1], sQ[ck - 1][cj], sQ[ck][cj], sQ[ck][cj - 1]};
      const double u0v = sU0[kk + 1][jj + 1], v0v = sV0[kk + 1][jj + 1];
      DivFast f;
      accelerate_node(f, rr, pp, qq, u0v, v0v, dx, dy, dt, uu, vv);
      if (f.bad) {
        DivIEEE x;
        accelerate_node(x, rr, pp, qq, u0v, v0v, dx, dy, dt, uu, vv);
      }
    }
    sU1[kk][jj] = uu; sV1[kk][jj] = vv;
  }
  __syncthreads();

  // PdV corrector + flux_calc (c.7) on the tile; write nodes/faces owned by
  // the tile (+ the last node/face row/column of the chunk).
  const int tj = threadIdx.x, tk = threadIdx.y;
  const int j = J0 + tj, k = K0 + tk;
  if (j <= c.nx && k <= c.ny) {
    const int cj = tj + 1, ck = tk + 1;   // ring cell index
    const int nj = tj + 1, nk = tk + 1;   // ring node index of node (j,k)
    const double ua = sU0[nk][nj], ub = sU0[nk + 1][nj], uc = sU0[nk][nj + 1], ud = sU0[nk + 1][nj + 1];
    const double va = sV0[nk][nj], vb = sV0[nk][nj + 1], vc = sV0[nk + 1][nj], vd = sV0[nk + 1][nj + 1];
    const double a1 = sU1[tk][tj], b1 = sU1[tk + 1][tj], c1 = sU1[tk][tj + 1], e1u = sU1[tk + 1][tj + 1];
    const double a1v = sV1[tk][tj], b1v = sV1[tk][tj + 1], c1v = sV1[tk + 1][tj], d1v = sV1[tk + 1][tj + 1];
    const double lsum = ua + ub + a1 + b1, rsum = uc + ud + c1 + e1u;
    const double bsum = va + vb + a1v + b1v, tsum = vc + vd + c1v + d1v;
    const double r = sR[ck][cj], e = sE[ck][cj], ph = sPh[ck][cj], qq = sQ[ck][cj];
    double ev, dvv;
    DivFast f;
    pdv_correct(f, r, e, ph, qq, lsum, rsum, bsum, tsum, dx, dy, dt, ev, dvv);
    if (f.bad) {
      DivIEEE x;
      pdv_correct(x, r, e, ph, qq, lsum, rsum, bsum, tsum, dx, dy, dt, ev, dvv);
    }
    store_field(c, e1, K_CELL, j, k, ev);
    store_field(c, d1, K_CELL, j, k, dvv);

    // flux_calc: x-face (j,k) and y-face (j,k); the chunk's last face
    // column/row is written by the cell next to it.
    const double cx = 0.25 * dt * dy, cy = 0.25 * dt * dx;
    store_field(c, fx, K_XFACE, j, k, cx * lsum);
    store_field(c, fy, K_YFACE, j, k, cy * bsum);
    if (j == c.nx) store_field(c, fx, K_XFACE, j + 1, k, cx * rsum);
    if (k == c.ny) store_field(c, fy, K_YFACE, j, k + 1, cy * tsum);

    // nodes
    store_field(c, u1, K_XVEL, j, k, a1);
    store_field(c, v1, K_YVEL, j, k, a1v);
    if (j == c.nx) {
      store_field(c, u1, K_XVEL, j + 1, k, c1);
      store_field(c, v1, K_YVEL, j + 1, k, b1v);
    }
    if (k == c.ny) {
      store_field(c, u1, K_XVEL, j, k + 1, b1);
      store_field(c, v1, K_YVEL, j, k + 1, c1v);
    }
    if (j == c.nx && k == c.ny) {
      store_field(c, u1, K_XVEL, j + 1, k + 1, e1u);
      store_field(c, v1, K_YVEL, j + 1, k + 1, d1v);
    }
  }
}

// ------------------------------------------------ advec_cell (c.8)
constexpr double ONE_BY_SIX = 1.0 / 6.0;

// Donor-cell flux with the limiter of c.8 for one face.  pv_don = pre_vol of
// the donor cell; r*/e* = density/energy at upwind, donor, downwind.
template <class D>
__device__ __forceinline__ void cell_face_flux(D& dv, double F, double pv_don, double ru, double rd,
                                               double rw, double eu, double ed, double ew,
                                               double& mflux, double& eflux) {
  double sigmat = dv(fabs(F), pv_don);
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
  double sigmam = dv(fabs(mflux), rd * pv_don);
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

constexpr int AX = 32, AY = 8;

// x sweep.  SWEEP 1: pre_vol = V + (dFx + dFy); SWEEP 2: pre_vol = V + dFx.
template <int SWEEP>
__global__ void __launch_bounds__(AX * AY)
k_advec_cell_x(Chunk c, const double* __restrict__ rho, const double* __restrict__ en,
               const double* __restrict__ fx, const double* __restrict__ fy,
               double* __restrict__ rho_out, double* __restrict__ en_out,
               double* __restrict__ mfx) {
  __shared__ double sM[AY][AX + 1], sEF[AY][AX + 1];
  const int J0 = blockIdx.x * AX + 1, K0 = blockIdx.y * AY + 1;
  const int tid = threadIdx.y * AX + threadIdx.x;
  const double vol = c.dx * c.dy;
  auto pre_vol = [&](int j, int k) -> double {
    const int i = idx(c, j, k);
    if (SWEEP == 1) return vol + (fx[i + 1] - fx[i] + fy[i + c.pitch] - fy[i]);
    return vol + fx[i + 1] - fx[i];
  };
  for (int t = tid; t < (AX + 1) * AY; t += AX * AY) {
    const int jj = t % (AX + 1), kk = t / (AX + 1);
    const int j = J0 + jj, k = K0 + kk;
    double m = 0.0, ef = 0.0;
    if (j <= c.nx + 1 && k <= c.ny) {
      const double F = fx[idx(c, j, k)];
      int up, don, dw;
      if (F > 0.0) {
        up = j - 2; don = j - 1; dw = j;
      } else {
        up = min(j + 1, c.nx + 2); don = j; dw = j - 1;
      }
      const int r0 = idx(c, 0, k);
      const double pv = pre_vol(don, k);
      const double ru = rho[r0 + up], rd = rho[r0 + don], rw = rho[r0 + dw];
      const double eu = en[r0 + up], ed = en[r0 + don], ew = en[r0 + dw];
      DivFast f;
      cell_face_flux(f, F, pv, ru, rd, rw, eu, ed, ew, m, ef);
      if (f.bad) {
        DivIEEE x;
        cell_face_flux(x, F, pv, ru, rd, rw, eu, ed, ew, m, ef);
      }
    }
    sM[kk][jj] = m; sEF[kk][jj] = ef;
  }
  __syncthreads();
  const int tj = threadIdx.x, tk = threadIdx.y;
  const int j = J0 + tj, k = K0 + tk;
  if (j <= c.nx && k <= c.ny) {
    const int i = idx(c, j, k);
    const double pv = pre_vol(j, k);
    const double rr = rho[i], ee = en[i], flo = fx[i], fhi = fx[i + 1];
    double ro, eo;
    DivFast f;
    cell_update(f, rr, ee, pv, sM[tk][tj], sM[tk][tj + 1], sEF[tk][tj], sEF[tk][tj + 1], flo, fhi, ro, eo);
    if (f.bad) {
      DivIEEE x;
      cell_update(x, rr, ee, pv, sM[tk][tj], sM[tk][tj + 1], sEF[tk][tj], sEF[tk][tj + 1], flo, fhi, ro, eo);
    }
    store_field(c, rho_out, K_CELL, j, k, ro);
    store_field(c, en_out, K_CELL, j, k, eo);
    store_field(c, mfx, K_XFACE, j, k, sM[tk][tj]);
    if (j == c.nx) store_field(c, mfx, K_XFACE, j + 1, k, sM[tk][tj + 1]);
  }
}

template <int SWEEP>
__global__ void __launch_bounds__(AX * AY)
k_advec_cell_y(Chunk c, const double* __restrict__ rho, const double* __restrict__ en,
               const double* __restrict__ fx, const double* __restrict__ fy,
               double* __restrict__ rho_out, double* __restrict__ en_out,
               double* __restrict__ mfy) {
  __shared__ double sM[AY + 1][AX], sEF[AY + 1][AX];
  const int J0 = blockIdx.x * AX + 1, K0 = blockIdx.y * AY + 1;
  const int tid = threadIdx.y * AX + threadIdx.x;
  const double vol = c.dx * c.dy;
  const int P = c.pitch;
  auto pre_vol = [&](int j, int k) -> double {
    const int i = idx(c, j, k);
    if (SWEEP == 1) return vol + (fy[i + P] - fy[i] + fx[i + 1] - fx[i]);
    return vol + fy[i + P] - fy[i];
  };
  for (int t = tid; t < AX * (AY + 1); t += AX * AY) {
    const int jj = t % AX, kk = t / AX;
    const int j = J0 + jj, k = K0 + kk;
    double m = 0.0, ef = 0.0;
    if (j <= c.nx && k <= c.ny + 1) {
      const double F = fy[idx(c, j, k)];
      int up, don, dw;
      if (F > 0.0) {
        up = k - 2; don = k - 1; dw = k;
      } else {
        up = min(k + 1, c.ny + 2); don = k; dw = k - 1;
      }
      const double pv = pre_vol(j, don);
      const double ru = rho[idx(c, j, up)], rd = rho[idx(c, j, don)], rw = rho[idx(c, j, dw)];
      const double eu = en[idx(c, j, up)], ed = en[idx(c, j, don)], ew = en[idx(c, j, dw)];
      DivFast f;
      cell_face_flux(f, F, pv, ru, rd, rw, eu, ed, ew, m, ef);
      if (f.bad) {
        DivIEEE x;
        cell_face_flux(x, F, pv, ru, rd, rw, eu, ed, ew, m, ef);
      }
    }
    sM[kk][jj] = m; sEF[kk][jj] = ef;
  }
  __syncthreads();
  const int tj = threadIdx.x, tk = threadIdx.y;
  const int j = J0 + tj, k = K0 + tk;
  if (j <= c.nx && k <= c.ny) {
    const int i = idx(c, j, k);
    const double pv = pre_vol(j, k);
    const double rr = rho[i], ee = en[i], flo = fy[i], fhi = fy[i + P];
    double ro, eo;
    DivFast f;
    cell_update(f, rr, ee, pv, sM[tk][tj], sM[tk + 1][tj], sEF[tk][tj], sEF[tk + 1][tj], flo, fhi, ro, eo);
    if (f.bad) {
      DivIEEE x;
      cell_update(x, rr, ee, pv, sM[tk][tj], sM[tk + 1][tj], sEF[tk][tj], sEF[tk + 1][tj], flo, fhi, ro, eo);
    }
    store_field(c, rho_out, K_CELL, j, k, ro);
    store_field(c, en_out, K_CELL, j, k, eo);
    store_field(c, mfy, K_YFACE, j, k, sM[tk][tj]);
    if (k == c.ny) store_field(c, mfy, K_YFACE, j, k + 1, sM[tk + 1][tj]);
  }
}

// ------------------------------------------------ advec_mom (c.9)
// Momentum flux at one node for one velocity component (limited, c.9).
template <class D>
__device__ __forceinline__ double mom_flux(D& dv, double nf, double nmp_don, double vup,
                                           double vdon, double vdw, double width, double cdif) {
  double sigma = dv(fabs(nf), nmp_don);
  double vdiffuw = vdon - vup;
  double vdiffdw = vdw - vdon;
  double limiter = 0.0;
  if (vdiffuw * vdiffdw > 0.0) {
    double auw = fabs(vdiffuw);
    double adw = fabs(vdiffdw);
    double wind = 1.0;
    if (vdiffdw <= 0.0) wind = -1.0;
    limiter = wind * fmin(fmin(dv(width * (dv((2.0 - sigma) * adw, width) +
                                           dv((1.0 + sigma) * auw, cdif)),
                                  6.0),
                               auw), adw);
  }
  double advec_vel = vdon + (1.0 - sigma) * limiter;
  return advec_vel * nf;
}

// both velocity components at one node (they share sigma's inputs)
template <class D>
__device__ __forceinline__ void mom_flux2(D& dv, double nf, double nmp, const double* uu,
                                          const double* vv, double w, double& mu, double& mv) {
  mu = mom_flux(dv, nf, nmp, uu[0], uu[1], uu[2], w, w);
  mv = mom_flux(dv, nf, nmp, vv[0], vv[1], vv[2], w, w);
}

template <class D>
__device__ __forceinline__ void mom_update(D& dv, double u, double v, double pre, double post,
                                           double mulo, double muhi, double mvlo, double mvhi,
                                           double& un, double& vn) {
  un = dv(u * pre + mulo - muhi, post);
  vn = dv(v * pre + mvlo - mvhi, post);
}

// x direction: nodes (j,k) j in [1,nx+1], k in [1,ny+1].  SWEEP 1 uses
// post_vol = V + dFy (mom_sweep 1), SWEEP 2 post_vol = V (mom_sweep 3).
template <int SWEEP>
__global__ void __launch_bounds__(AX * AY)
k_advec_mom_x(Chunk c, const double* __restrict__ rho, const double* __restrict__ mfx,
              const double* __restrict__ fy, const double* __restrict__ uin,
              const double* __restrict__ vin, double* __restrict__ uout,
              double* __restrict__ vout) {
  // node columns: nf on [J0-2, J0+AX] (AX+3), nmpost/nmp on [J0-1, J0+AX] (AX+2),
  // mom flux on [J0-1, J0+AX-1] (AX+1)
  constexpr int NF = AX + 3, NM = AX + 2, MF = AX + 1;
  __shared__ double sNF[AY][NF], sPost[AY][NM], sPre[AY][NM], sMU[AY][MF], sMV[AY][MF];
  const int J0 = blockIdx.x * AX + 1, K0 = blockIdx.y * AY + 1;
  const int tid = threadIdx.y * AX + threadIdx.x;
  const double vol = c.dx * c.dy;
  const int P = c.pitch;
  auto mass_post = [&](int i) -> double {  // rho*post_vol of cell at offset i
    const double pv = (SWEEP == 1) ? vol + fy[i + P] - fy[i] : vol;
    return rho[i] * pv;
  };
  for (int t = tid; t < NF * AY; t += AX * AY) {
    const int ii = t % NF, kk = t / NF;
    const int j = J0 - 2 + ii, k = K0 + kk;
    double nf = 0.0;
    if (j <= c.nx + 2 && k <= c.ny + 1) {
      const int i = idx(c, j, k);
      nf = 0.25 * (mfx[i - P] + mfx[i] + mfx[i + 1 - P] + mfx[i + 1]);
    }
    sNF[kk][ii] = nf;
  }
  for (int t = tid; t < NM * AY; t += AX * AY) {
    const int ii = t % NM, kk = t / NM;
    const int j = J0 - 1 + ii, k = K0 + kk;
    double post = 1.0;
    if (j <= c.nx + 2 && k <= c.ny + 1) {
      const int i = idx(c, j, k);
      post = 0.25 * (mass_post(i - P) + mass_post(i) + mass_post(i - 1 - P) + mass_post(i - 1));
    }
    sPost[kk][ii] = post;
  }
  __syncthreads();
  for (int t = tid; t < NM * AY; t += AX * AY) {
    const int ii = t % NM, kk = t / NM;
    // node j = J0-1+ii: nf(j-1) is sNF[ii], nf(j) is sNF[ii+1]
    sPre[kk][ii] = sPost[kk][ii] - sNF[kk][ii] + sNF[kk][ii + 1];
  }
  __syncthreads();
  for (int t = tid; t < MF * AY; t += AX * AY) {
    const int ii = t % MF, kk = t / MF;
    const int j = J0 - 1 + ii, k = K0 + kk;
    double mu = 0.0, mv = 0.0;
    if (j <= c.nx + 1 && k <= c.ny + 1) {
      const double nf = sNF[kk][ii + 1];  // nf(j)
      int up, don, dw;
      if (nf < 0.0) {
        up = j + 2; don = j + 1; dw = j;
      } else {
        up = j - 1; don = j; dw = j + 1;
      }
      const double nmp = sPre[kk][don - (J0 - 1)];
      const int r0 = idx(c, 0, k);
      const double uu[3] = {uin[r0 + up], uin[r0 + don], uin[r0 + dw]};
      const double vv[3] = {vin[r0 + up], vin[r0 + don], vin[r0 + dw]};
      DivFast f;
      mom_flux2(f, nf, nmp, uu, vv, c.dx, mu, mv);
      if (f.bad) {
        DivIEEE x;
        mom_flux2(x, nf, nmp, uu, vv, c.dx, mu, mv);
      }
    }
    sMU[kk][ii] = mu; sMV[kk][ii] = mv;
  }
  __syncthreads();
  const int tj = threadIdx.x, tk = threadIdx.y;
  const int j = J0 + tj, k = K0 + tk;
  if (j <= c.nx + 1 && k <= c.ny + 1) {
    const int i = idx(c, j, k);
    const double pre = sPre[tk][tj + 1], post = sPost[tk][tj + 1];
    const double u = uin[i], v = vin[i];
    double un, vn;
    DivFast f;
    mom_update(f, u, v, pre, post, sMU[tk][tj], sMU[tk][tj + 1], sMV[tk][tj], sMV[tk][tj + 1], un, vn);
    if (f.bad) {
      DivIEEE x;
      mom_update(x, u, v, pre, post, sMU[tk][tj], sMU[tk][tj + 1], sMV[tk][tj], sMV[tk][tj + 1], un, vn);
    }
    store_field(c, uout, K_XVEL, j, k, un);
    store_field(c, vout, K_YVEL, j, k, vn);
  }
}

// y direction: SWEEP 1 post_vol = V + dFx (mom_sweep 2), SWEEP 2 = V (4).
template <int SWEEP>
__global__ void __launch_bounds__(AX * AY)
k_advec_mom_y(Chunk c, const double* __restrict__ rho, const double* __restrict__ mfy,
              const double* __restrict__ fx, const double* __restrict__ uin,
              const double* __restrict__ vin, double* __restrict__ uout,
              double* __restrict__ vout) {
  constexpr int NF = AY + 3, NM = AY + 2, MF = AY + 1;
  __shared__ double sNF[NF][AX], sPost[NM][AX], sPre[NM][AX], sMU[MF][AX], sMV[MF][AX];
  const int J0 = blockIdx.x * AX + 1, K0 = blockIdx.y * AY + 1;
  const int tid = threadIdx.y * AX + threadIdx.x;
  const double vol = c.dx * c.dy;
  const int P = c.pitch;
  auto mass_post = [&](int i) -> double {
    const double pv = (SWEEP == 1) ? vol + fx[i + 1] - fx[i] : vol;
    return rho[i] * pv;
  };
  for (int t = tid; t < NF * AX; t += AX * AY) {
    const int jj = t % AX, ii = t / AX;
    const int j = J0 + jj, k = K0 - 2 + ii;
    double nf = 0.0;
    if (j <= c.nx + 1 && k <= c.ny + 2) {
      const int i = idx(c, j, k);
      nf = 0.25 * (mfy[i - 1] + mfy[i] + mfy[i - 1 + P] + mfy[i + P]);
    }
    sNF[ii][jj] = nf;
  }
  for (int t = tid; t < NM * AX; t += AX * AY) {
    const int jj = t % AX, ii = t / AX;
    const int j = J0 + jj, k = K0 - 1 + ii;
    double post = 1.0;
    if (j <= c.nx + 1 && k <= c.ny + 2) {
      const int i = idx(c, j, k);
      post = 0.25 * (mass_post(i - P) + mass_post(i) + mass_post(i - 1 - P) + mass_post(i - 1));
    }
    sPost[ii][jj] = post;
  }
  __syncthreads();
  for (int t = tid; t < NM * AX; t += AX * AY) {
    const int jj = t % AX, ii = t / AX;
    sPre[ii][jj] = sPost[ii][jj] - sNF[ii][jj] + sNF[ii + 1][jj];
  }
  __syncthreads();
  for (int t = tid; t < MF * AX; t += AX * AY) {
    const int jj = t % AX, ii = t / AX;
    const int j = J0 + jj, k = K0 - 1 + ii;
    double mu = 0.0, mv = 0.0;
    if (j <= c.nx + 1 && k <= c.ny + 1) {
      const double nf = sNF[ii + 1][jj];
      int up, don, dw;
      if (nf < 0.0) {
        up = k + 2; don = k + 1; dw = k;
      } else {
        up = k - 1; don = k; dw = k + 1;
      }
      const double nmp = sPre[don - (K0 - 1)][jj];
      const double uu[3] = {uin[idx(c, j, up)], uin[idx(c, j, don)], uin[idx(c, j, dw)]};
      const double vv[3] = {vin[idx(c, j, up)], vin[idx(c, j, don)], vin[idx(c, j, dw)]};
      DivFast f;
      mom_flux2(f, nf, nmp, uu, vv, c.dy, mu, mv);
      if (f.bad) {
        DivIEEE x;
        mom_flux2(x, nf, nmp, uu, vv, c.dy, mu, mv);
      }
    }
    sMU[ii][jj] = mu; sMV[ii][jj] = mv;
  }
  __syncthreads();
  const int tj = threadIdx.x, tk = threadIdx.y;
  const int j = J0 + tj, k = K0 + tk;
  if (j <= c.nx + 1 && k <= c.ny + 1) {
    const int i = idx(c, j, k);
    const double pre = sPre[tk + 1][tj], post = sPost[tk + 1][tj];
    const double u = uin[i], v = vin[i];
    double un, vn;
    DivFast f;
    mom_update(f, u, v, pre, post, sMU[tk][tj], sMU[tk + 1][tj], sMV[tk][tj], sMV[tk + 1][tj], un, vn);
    if (f.bad) {
      DivIEEE x;
      mom_update(x, u, v, pre, post, sMU[tk][tj], sMU[tk + 1][tj], sMV[tk][tj], sMV[tk + 1][tj], un, vn);
    }
    store_field(c, uout, K_XVEL, j, k, un);
    store_field(c, vout, K_YVEL, j, k, vn);
  }
}

}  // namespace clover
