// clover_aux.cuh -- initialisation, reflective-halo, EOS readback and
// field_summary kernels (untimed / on-demand parts of the path).
//
// generate_chunk / initialise_chunk: SURVEY.md 8(c) c.1 (geometry from the
// GLOBAL index, reading A13, so every decomposition paints identical bits).
// update_halo reflect: c.10.  field_summary: c.12, deterministic tiles.
#pragma once
#include "clover_common.cuh"
#include "clover_kernels.cuh"

namespace clover {

constexpr int MAX_STATES = 32;

struct DevState {
  double density, energy, xvel, yvel;
  int geometry;  // 1 rect, 2 circle, 3 point
  double xmin, xmax, ymin, ymax, radius;
};

struct StateList {
  int n;
  DevState s[MAX_STATES];
};

struct GlobalGeom {
  int NX, NY;          // global cells
  double xmin, ymin, dx, dy;
};

__device__ __forceinline__ double vertex_x(const GlobalGeom& g, int j) {
  return g.xmin + g.dx * (double)(j - 1);
}
__device__ __forceinline__ double vertex_y(const GlobalGeom& g, int k) {
  return g.ymin + g.dy * (double)(k - 1);
}

// Index of the last state (in painting order) that covers global cell
// (gj, gk); 0 = background.  Cells in [-1, N+2] are tested, as the
// reference paints its halo cells too.
__device__ int cell_state(const GlobalGeom& g, const StateList& sl, int gj, int gk) {
  int hit = 0;
  for (int s = 1; s < sl.n; ++s) {
    const DevState& st = sl.s[s];
    bool h = false;
    if (st.geometry == 1) {
      h = vertex_x(g, gj + 1) >= st.xmin && vertex_x(g, gj) < st.xmax &&
          vertex_y(g, gk + 1) >= st.ymin && vertex_y(g, gk) < st.ymax;
    } else if (st.geometry == 2) {
      const double cx = 0.5 * (vertex_x(g, gj) + vertex_x(g, gj + 1));
      const double cy = 0.5 * (vertex_y(g, gk) + vertex_y(g, gk + 1));
      const double r = sqrt((cx - st.xmin) * (cx - st.xmin) + (cy - st.ymin) * (cy - st.ymin));
      h = r <= st.radius;
    } else if (st.geometry == 3) {
      h = vertex_x(g, gj) == st.xmin && vertex_y(g, gk) == st.ymin;
    }
    if (h) hit = s;
  }
  return hit;
}

// Paint every local point whose global index is inside the global interior
// of its kind (cells [1,N], nodes [1,N+1]); physical-wall halos are filled
// afterwards by k_reflect.
__global__ void k_generate(Chunk c, GlobalGeom g, StateList sl, double* __restrict__ d0,
                           double* __restrict__ e0, double* __restrict__ u0,
                           double* __restrict__ v0) {
  const int j = blockIdx.x * blockDim.x + threadIdx.x - HALO;
  const int k = blockIdx.y * blockDim.y + threadIdx.y - HALO;
  if (j > c.nx + 1 + HALO || k > c.ny + 1 + HALO) return;
  const int gj = c.gj0 + j, gk = c.gk0 + k;
  const int i = idx(c, j, k);
  if (gj >= 1 && gj <= g.NX && gk >= 1 && gk <= g.NY && j <= c.nx + HALO && k <= c.ny + HALO) {
    const int s = cell_state(g, sl, gj, gk);
    d0[i] = sl.s[s].density;
    e0[i] = sl.s[s].energy;
  }
  if (gj >= 1 && gj <= g.NX + 1 && gk >= 1 && gk <= g.NY + 1) {
    int s = 0;
    for (int kk = gk - 1; kk <= gk; ++kk)
      for (int jj = gj - 1; jj <= gj; ++jj) s = max(s, cell_state(g, sl, jj, kk));
    u0[i] = sl.s[s].xvel;
    v0[i] = sl.s[s].yvel;
  }
}

// Reflective halo of one field (c.10) on the chunk's physical walls: every
// halo point is the composed x/y mirror image of an interior point.
__global__ void k_reflect(Chunk c, double* __restrict__ f, int kind) {
  const int j = blockIdx.x * blockDim.x + threadIdx.x - HALO;
  const int k = blockIdx.y * blockDim.y + threadIdx.y - HALO;
  if (j > c.nx + 1 + HALO || k > c.ny + 1 + HALO) return;
  const KindInfo ki = kind_info(kind, c.face_cc);
  auto src = [](int i, int n, int mode, int wlo, int whi, int& sgn_flip) -> int {
    sgn_flip = 0;
    if (mode == M_CELL) {
      if (wlo && i < 1) { sgn_flip = 1; return 1 - i; }
      if (whi && i > n) { sgn_flip = 1; return 2 * n + 1 - i; }
    } else if (mode == M_NODE) {
      if (wlo && i < 1) { sgn_flip = 1; return 2 - i; }
      if (whi && i > n + 1) { sgn_flip = 1; return 2 * n + 2 - i; }
    } else {
      if (wlo && i < 1) { sgn_flip = 1; return 2 - i; }
      if (whi && i > n) { sgn_flip = 1; return 2 * n - i; }
    }
    return i;
  };
  int fx, fy;
  const int js = src(j, c.nx, ki.mx, c.wl, c.wr, fx);
  const int ks = src(k, c.ny, ki.my, c.wb, c.wt, fy);
  if (!fx && !fy) return;
  double v = f[idx(c, js, ks)];
  if (fx && ki.sx < 0) v = -v;
  if (fy && ki.sy < 0) v = -v;
  f[idx(c, j, k)] = v;
}

// pressure / soundspeed readback: ideal_gas(density0, energy0) (c.2)
__global__ void k_eos_field(Chunk c, const double* __restrict__ d0, const double* __restrict__ e0,
                            double* __restrict__ out, int soundspeed) {
  const int j = blockIdx.x * blockDim.x + threadIdx.x + 1;
  const int k = blockIdx.y * blockDim.y + threadIdx.y + 1;
  if (j > c.nx || k > c.ny) return;
  const int i = idx(c, j, k);
  out[i] = soundspeed ? eos_soundspeed_ieee(d0[i], e0[i]) : eos_pressure(d0[i], e0[i]);
}

// field_summary (c.12): one 16x16 tile of cells per CTA (8 warps of two
// tile rows each).  Per-cell terms are reduced in a fixed order: a warp
// butterfly (__shfl_xor_sync, offsets 16..1; a+b and b+a round alike, so
// every lane holds the same bits), then the 8 warp sums in warp order by
// one thread; 5 partials per tile.  The tiles are aligned to the global
// index, so the bits do not depend on the decomposition.
constexpr int ST = 16;
__global__ void __launch_bounds__(ST * ST)
k_summary(Chunk c, const double* __restrict__ d0, const double* __restrict__ e0,
          const double* __restrict__ u0, const double* __restrict__ v0,
          double* __restrict__ partials) {
  __shared__ double red[5][ST * ST / 32];
  const int j = blockIdx.x * ST + threadIdx.x + 1;
  const int k = blockIdx.y * ST + threadIdx.y + 1;
  const int t = threadIdx.y * ST + threadIdx.x;
  double a[5] = {0.0, 0.0, 0.0, 0.0, 0.0};
  if (j <= c.nx && k <= c.ny) {
    const int i = idx(c, j, k);
    const int P = c.pitch;
    double vsqrd = 0.0;
    vsqrd = vsqrd + 0.25 * (u0[i] * u0[i] + v0[i] * v0[i]);
    vsqrd = vsqrd + 0.25 * (u0[i + 1] * u0[i + 1] + v0[i + 1] * v0[i + 1]);
    vsqrd = vsqrd + 0.25 * (u0[i + P] * u0[i + P] + v0[i + P] * v0[i + P]);
    vsqrd = vsqrd + 0.25 * (u0[i + P + 1] * u0[i + P + 1] + v0[i + P + 1] * v0[i + P + 1]);
    const double cell_vol = c.dx * c.dy;
    const double cell_mass = cell_vol * d0[i];
    a[0] = cell_vol;
    a[1] = cell_mass;
    a[2] = cell_mass * e0[i];
    a[3] = cell_mass * 0.5 * vsqrd;
    a[4] = cell_vol * eos_pressure(d0[i], e0[i]);
  }
#pragma unroll
  for (int q = 0; q < 5; ++q) {
    double x = a[q];
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) x = x + __shfl_xor_sync(0xffffffffu, x, o);
    if ((t & 31) == 0) red[q][t >> 5] = x;
  }
  __syncthreads();
  if (t < 5) {
    double x = red[t][0];
    for (int w = 1; w < ST * ST / 32; ++w) x = x + red[t][w];
    partials[((int64_t)blockIdx.y * gridDim.x + blockIdx.x) * 5 + t] = x;
  }
}

}  // namespace clover
