// clover_stream.cuh -- row-streaming sm_100a kernels of the CloverLeaf 2D
// step (the production path; clover_kernels.cuh holds the per-point math).
//
// Thread mapping: one thread per mesh column j, each
// thread walks a segment of rows k keeping the rows it still needs in
// registers, so every field element is loaded once per kernel and index
// arithmetic is one add per row.  Warps are 32 consecutive columns
// (coalesced 256-B row segments).  Neighbour values along x that are
// COMPUTED in the same kernel (half-step pressure, face fluxes, node masses,
// momentum fluxes) come from the adjacent lane via warp shuffles; the
// kernels whose x stencil reaches computed values overlap their warps by
// 1-3 "halo lanes".  Raw inputs at x-neighbours are plain L1-cached loads.
//
// All arithmetic is in the per-point functions of clover_kernels.cuh
// (evaluation order of SURVEY 8(c)).  Each kernel is a warp-segment body
// templated on the division policy.  The production launch runs it with
// DivFast (no IEEE code in the kernel at all); a warp whose sticky
// tiny-numerator flag is set pushes (warp, segment) onto a fix list, and a
// small fixup launch right after (kf_*) recomputes exactly those warp
// segments with IEEE division, overwriting the same outputs.  Every kernel
// is out-of-place, so the inputs are still intact for the redo.
#pragma once
#include "clover_common.cuh"
#include "clover_kernels.cuh"

namespace clover {

constexpr unsigned FULL = 0xffffffffu;
#ifndef CLOVER_SB
#define CLOVER_SB 32
#endif
constexpr int SB = CLOVER_SB;  // threads per block (one warp: a block slot frees as soon as its
                               // warp's segment is done; measured faster than 2-warp blocks for the
                               // Lagrangian and both sweeps)
#ifndef CLOVER_SBV
#define CLOVER_SBV 32
#endif
constexpr int SBV = CLOVER_SBV;  // visc_dt threads per block (64 was faster on the bm window with
                                 // 1-row ring slots; with 4-row slots 32 is as fast there and 5 %
                                 // faster on active flow: profiles/r2_sbv_box_ab.jsonl)

// Tunables (defaults = measured best; scripts/ab_variants.py builds others).
#define CLOVER_STR2(x) #x
#define CLOVER_STR(x) CLOVER_STR2(x)
#ifdef CLOVER_UNROLL  // default: the compiler's own unrolling (measured best)
#define STREAM_LOOP _Pragma(CLOVER_STR(unroll CLOVER_UNROLL))
#else
#define STREAM_LOOP
#endif
// min resident blocks/SM (register cap) for visc_dt+lagrangian / advection;
// 0 = plain __launch_bounds__(SB) (ptxas heuristic).  Measured on B200 at
// 3840^2 (scripts/ab_variants.py), 64-thread blocks: lagrangian 10 (96 regs),
// visc_dt uncapped, advection 16 (64 regs), mom_y 14.  Short row segments
// (8-16 rows) measured 6 % faster than 16-32 (more, shorter blocks).
// Round 2, 32-thread blocks: the Lagrangian at (32, 10), which ptxas
// compiles to 108 registers (18 warps/SM: 0.262 -> 0.253 ms; plain (32)
// gives 80), the unfused advection kernels at the same warps per SM as
// before (the counts scale with 64 / SB).
#ifndef CLOVER_MINB_HEAVY
#define CLOVER_MINB_HEAVY 10
#endif
#ifndef CLOVER_MINB_ADV
#define CLOVER_MINB_ADV (16 * 64 / CLOVER_SB)
#endif
#ifndef CLOVER_MINB_VISC
#define CLOVER_MINB_VISC 0
#endif
#ifndef CLOVER_MINB_ADVX
#define CLOVER_MINB_ADVX 0
#endif
#if CLOVER_MINB_ADVX > 0
#define LB_ADVX __launch_bounds__(SB, CLOVER_MINB_ADVX)
#else
#define LB_ADVX __launch_bounds__(SB)
#endif
#ifndef CLOVER_MINB_ADVY
#define CLOVER_MINB_ADVY 0
#endif
#if CLOVER_MINB_ADVY > 0
#define LB_ADVY __launch_bounds__(SB, CLOVER_MINB_ADVY)
#else
#define LB_ADVY __launch_bounds__(SB)
#endif
#ifndef CLOVER_MINB_MOMY
#define CLOVER_MINB_MOMY (14 * 64 / CLOVER_SB)
#endif
#if CLOVER_MINB_MOMY > 0
#define LB_MOMY __launch_bounds__(SB, CLOVER_MINB_MOMY)
#else
#define LB_MOMY __launch_bounds__(SB)
#endif
#if CLOVER_MINB_HEAVY > 0
#define LB_HEAVY __launch_bounds__(SB, CLOVER_MINB_HEAVY)
#else
#define LB_HEAVY __launch_bounds__(SB)
#endif
#if CLOVER_MINB_VISC > 0
#define LB_VISC __launch_bounds__(SBV, CLOVER_MINB_VISC)
#else
#define LB_VISC __launch_bounds__(SBV)
#endif
#if CLOVER_MINB_ADV > 0
#define LB_ADV __launch_bounds__(SB, CLOVER_MINB_ADV)
#else
#define LB_ADV __launch_bounds__(SB)
#endif
#ifndef CLOVER_VKS
#define CLOVER_VKS 32
#endif
#ifndef CLOVER_LKS
#define CLOVER_LKS 16
#endif
#ifndef CLOVER_CKS
#define CLOVER_CKS 8
#endif
#ifndef CLOVER_CKS_Y
#define CLOVER_CKS_Y 8
#endif
#ifndef CLOVER_MKS
#define CLOVER_MKS 8
#endif
#ifndef CLOVER_MKS_Y
#define CLOVER_MKS_Y 8
#endif

// Proxy fence before a ring slot is refilled.  The slot's shared-memory
// reads (generic proxy) are all consumed by arithmetic earlier in the same
// iteration and the warp is converged (__syncwarp) before lane 0 issues the
// TMA write, the same execution ordering CUTLASS's TMA pipelines rely on
// for the consumer release (mbarrier arrive, no proxy fence); the fence is
// kept as an option.  Measured at 3840^2: 0.5 % per step without it.
#ifndef CLOVER_TMA_RELEASE_FENCE
#define CLOVER_TMA_RELEASE_FENCE 0
#endif

// ---------------------------------------------------------------- fix lists
// hdr[0] = number of entries, hdr[1] = finished fixup blocks, hdr[2] =
// entries fixed so far (debug counter); e[] = (global
// warp, segment) of every warp whose fast pass flagged.  Capacity = warps
// of the fast grid (each warp pushes at most once), sized by the engine.
struct FixSlot {
  unsigned* hdr;
  uint2* e;
};
__device__ __forceinline__ void fix_push(FixSlot f, int lane, unsigned gw, unsigned seg) {
  if (lane == 0) {
    const unsigned n = atomicAdd(f.hdr, 1u);
    f.e[n] = make_uint2(gw, seg);
  }
}
// Fixup driver: every flagged segment (seg_rows_of) is redone one row per warp
// (row-parallel, so the fixup's latency is one row, not one segment); the
// last block to finish resets the list.  run(gw, k0, k1, lane, w) with
// k1 = k0 + 1; rows at or beyond `lim` are skipped.
struct NoLast {
  __device__ void operator()() const {}
};
// Fixup blocks (one warp each since the blocks have one warp: six per SM;
// 148 -> 444 warps redo the flagged rows, bm 3840^2 step 0.858 -> 0.847 ms,
// profiles/r2_fixblocks_ab.jsonl; 888 for the late steps, where 25-76
// segments a step are flagged: 300-step run 0.871 -> 0.868 ms,
// profiles/r2_fixblocks_full_ab.txt); a launch may add y-wall blocks.
#ifndef CLOVER_FIX_BLOCKS
#define CLOVER_FIX_BLOCKS 888
#endif
constexpr int FIX_BLOCKS = CLOVER_FIX_BLOCKS;
template <int BS = SB, class Run, class Last = NoLast>
__device__ __forceinline__ void fix_loop(FixSlot f, int ks, int nb, int ch, int cf, int td, int lim, Run&& run,
                                         Last last = {}) {
  const unsigned n = *(volatile unsigned*)f.hdr;  // the same value in every thread
  if (n == 0u) {
    // nothing flagged (the common case): no list to reset, no counting
    if (blockIdx.x == 0 && threadIdx.x == 0) last();
    return;
  }
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  const unsigned items = n * (unsigned)ks;
  for (unsigned it = blockIdx.x * (BS / 32) + w; it < items; it += FIX_BLOCKS * (BS / 32)) {
    const uint2 t = f.e[it / ks];
    int ks0, len;
    seg_rows_lay((int)t.y, ks, nb, ch, cf, lim - 1, ks0, len, td);
    const int r = (int)(it % ks);
    const int k0 = ks0 + r;
    if (r < len && k0 < lim) run((int)t.x, k0, k0 + 1, lane, w);
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    __threadfence();
    if (atomicAdd(f.hdr + 1, 1u) == FIX_BLOCKS - 1) {
      f.hdr[2] += n;  // cumulative (clover_debug_fix_count)
      __threadfence();  // every block's fixes before the reset (y_walls_after_fix waits on it)
      f.hdr[0] = 0u;
      f.hdr[1] = 0u;
      __threadfence();
      last();  // runs after every block's work (and atomics) of this launch
    }
  }
}

// ---------------------------------------------------------------- y-wall bands
// advec_cell y on the wall bands (cell rows 1..3 and ny-1..ny, IEEE
// division: bitwise the fast path's results) so the fused y sweep finds
// the mirrored halo rows of the post-sweep density and the y-face mass flux.
// One thread per (column, band row): the five band rows are independent --
// each thread evaluates the two faces of its cell with the expressions the
// row-streaming body (advec_cell_y_body) uses, -fmad=false: same bits -- so
// the band's latency is one row's division chain.  Halo columns at x chunk
// boundaries too: the fused y sweep's halo lanes recompute their interior
// rows but read these wall rows.
struct YWalls {
  int nbx;  // blocks per band row (0: no wall work in this launch)
  const double *rho, *en, *fx, *fy;
  double *rho_out, *en_out, *mfy;
};
template <int SWEEP>
__device__ __forceinline__ void y_walls_block(const Chunk& c, const YWalls& y, int bx, int b) {
  const int k = b < 3 ? 1 + b : c.ny - 4 + b;
  if (b < 3 && k > c.ny) return;
  if (b < 3 ? !c.wb : !c.wt) return;  // a chunk boundary: the y sweep recomputes these rows
  const int jlo = c.wl ? 1 : 0;
  Chunk cw = c;
  cw.nx = c.wr ? c.nx : c.nx + 1;
  const int j = bx * SB + threadIdx.x + jlo;
  if (j > cw.nx) return;
  const double* __restrict__ rho = y.rho;
  const double* __restrict__ en = y.en;
  const double* __restrict__ fx = y.fx;
  const double* __restrict__ fy = y.fy;
  DivIEEE dv;
  const double vol = cw.dx * cw.dy;
  const int P = cw.pitch;
  auto pre_vol = [&](int i) -> double {
    if (SWEEP == 1) return vol + (fy[i + P] - fy[i] + fx[i + 1] - fx[i]);
    return vol + fy[i + P] - fy[i];
  };
  const int i = idx(cw, j, k);
  const double R0 = rho[i - 2 * P], R1 = rho[i - P], R2 = rho[i], R3 = rho[i + P],
               R4 = rho[i + 2 * P];
  const double E0 = en[i - 2 * P], E1 = en[i - P], E2 = en[i], E3 = en[i + P], E4 = en[i + 2 * P];
  const double pvm = pre_vol(i - P), pv0 = pre_vol(i), pv1 = pre_vol(i + P);
  double m0, ef0, m1, ef1;
  {  // face k
    const double F = fy[i];
    if (F > 0.0) cell_face_flux(dv, F, pvm, R0, R1, R2, E0, E1, E2, m0, ef0);
    else cell_face_flux(dv, F, pv0, R3, R2, R1, E3, E2, E1, m0, ef0);
  }
  {  // face k+1
    const double F = fy[i + P];
    if (F > 0.0) cell_face_flux(dv, F, pv0, R1, R2, R3, E1, E2, E3, m1, ef1);
    else cell_face_flux(dv, F, pv1, R4, R3, R2, E4, E3, E2, m1, ef1);
  }
  double ro, eo;
  cell_update(dv, R2, E2, pv0, m0, m1, ef0, ef1, fy[i], fy[i + P], ro, eo);
  const bool near = near_wall_col(cw, j) || near_wall_row(cw, k);
  store_at(cw, y.rho_out, K_CELL, j, k, i, near, ro);
  store_at(cw, y.en_out, K_CELL, j, k, i, near, eo);
  store_at(cw, y.mfy, K_YFACE, j, k, i, near, m0);
  if (k == cw.ny) store_field(cw, y.mfy, K_YFACE, j, k + 1, m1);
}
// The wall bands carried by the fixup launch that precedes the y sweep (one
// chunk on one rank: one launch hop fewer per step).  Blocks FIX_BLOCKS..
// wait until the fixups of the previous kernel are done (fix_loop's last
// block resets hdr[0] after a fence; 0 from the start when nothing was
// flagged, the common case), then compute the bands.  Every block of the
// launch is co-resident (small blocks), so the wait cannot starve the fixups.
template <int SWEEP>
__device__ __forceinline__ bool y_walls_after_fix(const Chunk& c, FixSlot f, const YWalls& y) {
  if ((int)blockIdx.x < FIX_BLOCKS) return false;
  if (threadIdx.x == 0) {
    unsigned v;
    for (;;) {
      asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(f.hdr) : "memory");
      if (v == 0u) break;
      __nanosleep(64);
    }
  }
  __syncthreads();
  const int b = (int)blockIdx.x - FIX_BLOCKS;
  y_walls_block<SWEEP>(c, y, b % y.nbx, b / y.nbx);
  return true;
}

// ================================================================ visc_dt
// Warp w of the grid owns columns j = 32*w + lane + 1 over rows [k0, k0+VKS).
// Rows of d0, e0, u0, v0 stream through a per-warp shared-memory ring of
// VSTG slots of VBOX rows, one 3D TMA tensor copy per slot (the four fields are consecutive
// equally spaced buffers); smem column t of a slot holds memory column
// COL0 - 1 + 32*w + t, so lane l reads its column at t = l+2 and both x
// neighbours.  Iteration k reads rows k and k+1 (the pressures of rows k-1
// and k are carried), then releases row k.  The box starts on an even
// column: a tensor copy of fp64 rows must start 16-B aligned in global
// memory (an odd start column faults with an illegal instruction on B200;
// scripts/tma_probe.cu).
constexpr int VKS = CLOVER_VKS;
#ifndef CLOVER_VSTG  // ring slots (boxes of VBOX rows)
#define CLOVER_VSTG 2
#endif
constexpr int VSTG = CLOVER_VSTG;
constexpr int VRW = 36;
// rows per tensor copy (ring slot): one copy brings VBOX consecutive rows of
// the four fields (box {VRW, VBOX, 4}; smem slot [field][row][column]).
// Round 2: 2 slots of 4 rows instead of 4 slots of 1 row -- the same
// bytes in flight in a quarter of the copies: bm window 0.136 -> 0.127 ms
// (profiles/r2_vbox_ab.jsonl; 2x4 and 3x2 rows 0.130 / 0.133, 2x8 0.145,
// 3x4 0.134); the kernel streams more than it computes there, and fewer,
// larger copies reach the data sooner.
#ifndef CLOVER_VBOX
#define CLOVER_VBOX 4
#endif
constexpr int VBOX = CLOVER_VBOX;
enum { VF_R, VF_E, VF_U, VF_V, VNF };  // = buffer order B_D0 B_E0 B_U0 B_V0
constexpr int VFS = VBOX * VRW;        // field stride in a slot (doubles)
constexpr int VSLOT = VNF * VFS;       // 1152 B per row: a multiple of 128 B
constexpr unsigned VBYTES = VNF * VFS * 8;
static_assert((VSLOT * 8) % 128 == 0 && VSTG >= 2, "visc ring");
static_assert(COL0 % 2 == 1, "visc ring box starts on an even (16-B aligned) column");

// Warp segment: columns j = 32*gw + lane + 1, rows [k0, k1).
// Returns whether any lane flagged; dtw = the warp's dt minimum (all lanes).
// EDGE = false: columns, their x neighbours and rows k0-1 .. k1 are at least
// HALO+2 away from every wall and chunk edge (visc_interior).
template <class D, bool EDGE>
__device__ __forceinline__ bool visc_body(const Chunk& c, const CUtensorMap* __restrict__ tm,
                                          double* __restrict__ q, const DtParams& prm, int gw,
                                          int k0, int k1, int lane, double* ring,
                                          unsigned long long* bars, double& dtw) {
  const int j = gw * 32 + lane + 1;
  double dtl = G_BIG;
  D dv;
  const int r_first = k0 - 1, r_last = k1;
  const int xcol = COL0 - 1 + gw * 32;  // even (COL0 = 15)
  // ring slot of a row: its box (VBOX rows from r_first) modulo VSTG
  auto slot_of = [&](int r) { return ((unsigned)(r - r_first) / (unsigned)VBOX) % (unsigned)VSTG; };
  auto issue = [&](int r) {  // the box whose first row is r
    const unsigned sl = slot_of(r);
    mbar_arrive_expect_tx(&bars[sl], VBYTES);
    tma_load_3d(ring + sl * VSLOT, tm, xcol, c.row0 + r, 0, &bars[sl]);
  };
  auto wait_row = [&](int r) {
    const unsigned box = (unsigned)(r - r_first) / (unsigned)VBOX;
    mbar_wait(&bars[box % VSTG], (box / VSTG) & 1u);
  };
  auto row = [&](int r) -> const double* {
    return ring + slot_of(r) * VSLOT + ((unsigned)(r - r_first) % (unsigned)VBOX) * VRW + lane + 2;
  };
  // row r consumed: when it is its box's last row, refill the slot with the
  // box VSTG boxes further on
  auto release = [&](int r) {
    const unsigned rel = (unsigned)(r - r_first);
    if (rel % VBOX == VBOX - 1 && lane == 0) {
      const int nr = r + 1 + (VSTG - 1) * VBOX;
      if (nr <= r_last) issue(nr);
    }
  };
  if (lane == 0) {
    for (int t = 0; t < VSTG; ++t) mbar_init(&bars[t], 1);
    fence_mbar_init();
    fence_proxy_async();
    for (int r = r_first; r < r_first + VSTG * VBOX && r <= r_last; r += VBOX) issue(r);
  }
  __syncwarp();
  const bool ncol = EDGE && near_wall_col(c, j);
  wait_row(r_first);
  wait_row(k0);
  double pcm = eos_pressure(row(r_first)[VF_R * VFS], row(r_first)[VF_E * VFS]);  // p(k-1)
  double pc = eos_pressure(row(k0)[VF_R * VFS], row(k0)[VF_E * VFS]);            // p(k)
#if CLOVER_TMA_RELEASE_FENCE
  fence_proxy_async();
#endif
  __syncwarp();
  release(r_first);  // row k0-1 is consumed
  DtAcc acc;
  // rows 0 / ny+1 at a y chunk boundary are ring rows (q only, no dt): the
  // Lagrangian phase reads q on ring 1, so no q exchange is needed in y
  if ((!EDGE || j <= c.nx) && k1 > k0 && (!EDGE || k0 >= 1))
    acc.bottom(row(k0)[VF_V * VFS], row(k0)[VF_V * VFS + 1], c);
  const bool left = EDGE && j == 1;  // column 1: no left neighbour takes this face
  int i = idx(c, j, k0);
  // (ring slots by mask: VSTG is a power of two; rotating the row pointers
  // as the Lagrangian and y-sweep bodies do measured neutral here, +2 regs)
  for (int k = k0; k < k1; ++k, i += c.pitch) {
    wait_row(k + 1);
    const double* rc = row(k);
    const double* rn = row(k + 1);
    const bool owned_row = !EDGE || (k >= 1 && k <= c.ny);
    if (!EDGE || j <= c.nx) {
      ViscIn I;
      I.rho = rc[VF_R * VFS]; I.e = rc[VF_E * VFS];
      I.pb = pcm;
      I.pt = eos_pressure(rn[VF_R * VFS], rn[VF_E * VFS]);
      I.pl = eos_pressure(rc[VF_R * VFS - 1], rc[VF_E * VFS - 1]);
      I.pr = eos_pressure(rc[VF_R * VFS + 1], rc[VF_E * VFS + 1]);
      I.u00 = rc[VF_U * VFS]; I.u10 = rc[VF_U * VFS + 1];
      I.u01 = rn[VF_U * VFS]; I.u11 = rn[VF_U * VFS + 1];
      I.v00 = rc[VF_V * VFS]; I.v10 = rc[VF_V * VFS + 1];
      I.v01 = rn[VF_V * VFS]; I.v11 = rn[VF_V * VFS + 1];
      double qv, cc2, c2;
      visc_cell(dv, I, c, qv, cc2, c2);
      if (owned_row) {
        if (EDGE && k == 1 && k0 == 0) acc.bottom(I.v00, I.v10, c);  // after ring row 0
        acc.add(I, c, qv, cc2, c2, left);
      }
      store_at(c, q, K_CELL, j, k, i, EDGE && (ncol || near_wall_row(c, k)), qv);
      pcm = pc;
      pc = I.pt;
    }
    // row k is consumed (row k+1 is read again next iteration): refill
#if CLOVER_TMA_RELEASE_FENCE
    fence_proxy_async();
#endif
    __syncwarp();
    release(k);
  }
  __syncwarp();
  if (lane == 0)
    for (int t = 0; t < VSTG; ++t) mbar_inval(&bars[t]);  // the ring may be reused (fixup)
  __syncwarp();
  if ((!EDGE || j <= c.nx) && k1 > k0) dtl = acc.dt(c, prm);
  for (int o = 16; o > 0; o >>= 1) dtl = fmin(dtl, __shfl_xor_sync(FULL, dtl, o));
  dtw = dtl;
  return __any_sync(FULL, dv.bad);
}

__device__ __forceinline__ bool visc_interior(const Chunk& c, int gw, int k0, int k1) {
  return gw * 32 >= HALO + 2 && gw * 32 + 34 <= c.nx - HALO - 1 && k0 - 1 >= HALO + 2 &&
         k1 <= c.ny - HALO - 1;
}

template <class D>
__device__ __forceinline__ bool visc_seg(const Chunk& c, const CUtensorMap* __restrict__ tm,
                                         double* __restrict__ q, const DtParams& prm, int gw,
                                         int k0, int k1, int lane, double* ring,
                                         unsigned long long* bars, double& dtw) {
  if (visc_interior(c, gw, k0, k1))
    return visc_body<D, false>(c, tm, q, prm, gw, k0, k1, lane, ring, bars, dtw);
  return visc_body<D, true>(c, tm, q, prm, gw, k0, k1, lane, ring, bars, dtw);
}

// Rows [k0, k1) of a visc segment extended by the ring row 0 (ny+1) when the
// segment starts at row 1 (ends at row ny) next to a y chunk boundary.
__device__ __forceinline__ void visc_ring_rows(const Chunk& c, int& k0, int& k1) {
  if (k0 == 1 && !c.wb) k0 = 0;
  if (k1 == c.ny + 1 && !c.wt) k1 = c.ny + 2;
}

__global__ void LB_VISC
ks_visc_dt(Chunk c, const __grid_constant__ CUtensorMap tm, double* __restrict__ q,
           StepScalars* __restrict__ s, DtParams prm, FixSlot fix) {
  pdl_trigger();
  pdl_wait();
  __shared__ __align__(128) double ring[SBV / 32][VSTG * VSLOT];
  __shared__ __align__(8) unsigned long long bars[SBV / 32][VSTG];
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const int gw = blockIdx.x * (SBV / 32) + warp;
  double dtw = G_BIG;
  int k0, len;
  const int sg = seg_y(c);
  seg_rows_lay(sg, c.vks, c.vnb, c.vch, c.vcf, c.ny, k0, len, c.vtd);
  if (len <= 0) return;  // empty band segment
  int k1 = min(k0 + len, c.ny + 1);
  visc_ring_rows(c, k0, k1);
  if (gw * 32 < c.nx) {
    if (visc_seg<DivFast>(c, &tm, q, prm, gw, k0, k1, lane, ring[warp], bars[warp], dtw)) {
      fix_push(fix, lane, gw, (unsigned)sg);
      dtw = G_BIG;  // this warp's dt comes from the fixup
    }
  }
  __shared__ double wmin[SBV / 32];
  if (lane == 0) wmin[warp] = dtw;
  __syncthreads();
  if (threadIdx.x == 0) {
    double m = wmin[0];
    for (int w = 1; w < SBV / 32; ++w) m = fmin(m, wmin[w]);
    dt_slot_min(s, m);
  }
}

__global__ void __launch_bounds__(SBV)
kf_visc_dt(Chunk c, const __grid_constant__ CUtensorMap tm, double* __restrict__ q,
           StepScalars* __restrict__ s, DtParams prm, FixSlot fix, double* __restrict__ hist,
           int fin) {
  pdl_trigger();
  pdl_wait();
  __shared__ __align__(128) double ring[SBV / 32][VSTG * VSLOT];
  __shared__ __align__(8) unsigned long long bars[SBV / 32][VSTG];
  // fin: single chunk on one rank -- the last block also finalises dt
  // (k_dt_finalize's work, once every contribution to the slot is in)
  fix_loop<SBV>(
      fix, c.vks, c.vnb, c.vch, c.vcf, c.vtd, c.ny + 1,
      [&](int gw, int k0, int k1, int lane, int w) {
        double dtw;
        visc_ring_rows(c, k0, k1);  // rows 1 / ny redo their ring row too
        visc_seg<DivIEEE>(c, &tm, q, prm, gw, k0, k1, lane, ring[w], bars[w], dtw);
        if (lane == 0) dt_slot_min(s, dtw);
      },
      [&]() {
        if (fin) dt_finalize(s, hist, prm);
      });
}

// ================================================================ Lagrangian
// Warp strip: lane l <-> column j = J0 - 1 + l, J0 = 1 + 30 * (global warp);
// lanes 1..30 own cells/nodes j (lane 0 and 31 are halo lanes).  Rows are
// streamed k = k0-1 .. k1: at row k the thread computes the PdV predictor +
// EOS of cell (j,k), accelerate at node (j,k) and the PdV corrector +
// flux_calc of cell (j,k-1).  Reflective walls: the half-step pressure of a
// ring cell outside the mesh is the mirror of the computed interior value
// (rows: recomputed from the mirrored row; columns: taken from the mirrored
// lane), exactly the reference's update_halo{pressure} after the predictor.
constexpr int LW = 30;   // owned columns per warp
static_assert((COL0 - 1 + LW) % 2 == 0 && LW % 2 == 0, "Lagrangian ring box starts on an even column");
constexpr int LKS = CLOVER_LKS;  // rows per segment

#ifndef CLOVER_LSTG
#define CLOVER_LSTG 6
#endif
// TMA-staged rows: one 3D tensor copy per mesh row brings the row segment of
// all five inputs (the engine keeps d0, e0, u0, v0, q as consecutive,
// equally spaced buffers: tensor dims {pitch, rows, field}) into a per-warp
// LSTG-row shared-memory ring, so the DRAM latency of row k+LSTG-2 overlaps
// the compute of row k.  Smem column t of a slot holds memory column
// COL0 + J0 - 2 + t: lane l reads its own column at t = l+1 and both x
// neighbours without shuffles.  Iteration k reads rows k-1, k and k+1 from
// the ring (raw inputs are never carried in registers), then releases row
// k-1's slot.
constexpr int LSTG = CLOVER_LSTG;  // ring rows
constexpr int LRW = 36;            // staged columns (>= 34, 16-B multiple)
enum { LF_R, LF_E, LF_U, LF_V, LF_Q, LNF };  // = buffer order B_D0 B_E0 B_U0 B_V0 B_Q
// rows per tensor copy (ring slot), as for visc_dt (VBOX): box {LRW, LBOX, 5},
// smem slot [field][row][column]
#ifndef CLOVER_LBOX
#define CLOVER_LBOX 1
#endif
constexpr int LBOX = CLOVER_LBOX;
constexpr int LFS = LBOX * LRW;    // field stride in a slot (doubles)
constexpr int LSLOT = (LNF * LFS + 15) / 16 * 16;  // doubles per slot, padded to 128 B (192 at LBOX 1)
constexpr unsigned LBYTES = LNF * LFS * 8;
static_assert(LSLOT >= LNF * LFS && (LSLOT * 8) % 128 == 0, "slot");
static_assert(LSTG >= 3, "ring");

// EDGE = false: a warp segment whose stencil reach is at least HALO+2 away
// from every wall and chunk edge (lagr_interior): constant lane predicates,
// no wall rows, no mirrored or extra stores.
template <class D, bool EDGE>
__device__ __forceinline__ bool lagr_body(const Chunk& c, const CUtensorMap* __restrict__ tm,
                                          double* __restrict__ d1, double* __restrict__ e1,
                                          double* __restrict__ u1, double* __restrict__ v1,
                                          double* __restrict__ fx, double* __restrict__ fy,
                                          const StepScalars* __restrict__ s, int gw, int k0,
                                          int k1, int lane, double* ring,
                                          unsigned long long* bars) {
  const int J0 = 1 + LW * gw;
  const int j = J0 - 1 + lane;
  if (J0 > c.nx) return false;  // whole warp beyond the chunk (rings are per warp)
  D dv;
  const double dt = s->dt, dx = c.dx, dy = c.dy;
  const bool colok = !EDGE || j <= c.nx + 1;
  const bool ncol = EDGE && near_wall_col(c, j);
  int src = lane;
  if (EDGE && c.wl && j == 0) src = lane + 1;
  if (EDGE && c.wr && j == c.nx + 1) src = lane - 1;
  const bool xwall_warp = EDGE && __any_sync(FULL, src != lane);

  const int r_first = k0 - 1, r_last = k1 + 1;  // staged rows
  const int xcol = COL0 + J0 - 2;  // = 14 + 30*gw: even, 16-B aligned (see visc_body)
  auto slot_of = [&](int r) { return ((unsigned)(r - r_first) / (unsigned)LBOX) % (unsigned)LSTG; };
  auto issue_at = [&](unsigned sl, int r) {  // row r into slot sl
    mbar_arrive_expect_tx(&bars[sl], LBYTES);
    tma_load_3d(ring + sl * LSLOT, tm, xcol, c.row0 + r, 0, &bars[sl]);
  };
  auto issue = [&](int r) { issue_at(slot_of(r), r); };
  auto wait_row = [&](int r) {
    const unsigned box = (unsigned)(r - r_first) / (unsigned)LBOX;
    mbar_wait(&bars[box % LSTG], (box / LSTG) & 1u);
  };
  auto row = [&](int r) -> const double* {
    return ring + slot_of(r) * LSLOT + ((unsigned)(r - r_first) % (unsigned)LBOX) * LRW + lane + 1;
  };
  // PdV predictor + EOS of the cell in row rc, node rows rc and rn (c.5)
  auto predict = [&](const double* rc, const double* rn) -> double {
    return pdv_predict_pressure(dv, rc[LF_R * LFS], rc[LF_E * LFS], rc[LF_Q * LFS],
                                rc[LF_U * LFS], rn[LF_U * LFS], rc[LF_U * LFS + 1],
                                rn[LF_U * LFS + 1], rc[LF_V * LFS], rc[LF_V * LFS + 1],
                                rn[LF_V * LFS], rn[LF_V * LFS + 1], dx, dy, c.rvol, dt);
  };
  if (lane == 0) {
    for (int t = 0; t < LSTG; ++t) mbar_init(&bars[t], 1);
    fence_mbar_init();
    fence_proxy_async();
    for (int r = r_first; r < r_first + LSTG * LBOX && r <= r_last; r += LBOX) issue(r);
  }
  __syncwarp();

  // row k0-1: half-step pressure only.  At a reflective bottom wall the
  // ring row 0 takes the mirror of row 1 (update_halo{pressure}), which is
  // the predictor evaluated on row 1's inputs.
  double ph_m, phl_m;
  // interior body: the predictor's top y-face flux of row k is the bottom
  // one of row k+1 (same expression, same node velocities): carried
  double tfp = 0.0;
  {
    const int kp = (EDGE && c.wb && k0 == 1) ? 1 : k0 - 1;
    for (int r = r_first; r <= kp + 1; ++r) wait_row(r);
    double ph = 0.0;
    if constexpr (EDGE) {
      if (colok) ph = predict(row(kp), row(kp + 1));
    } else {
      const double* a = row(kp);
      const double* b = row(kp + 1);
      tfp = pdv_face_pred(b[LF_V * LFS], b[LF_V * LFS + 1], dx, dt);
      ph = pdv_predict_pressure_bt(dv, a[LF_R * LFS], a[LF_E * LFS], a[LF_Q * LFS], a[LF_U * LFS],
                                   b[LF_U * LFS], a[LF_U * LFS + 1], b[LF_U * LFS + 1],
                                   pdv_face_pred(a[LF_V * LFS], a[LF_V * LFS + 1], dx, dt), tfp,
                                   dx, dy, c.rvol, dt);
    }
    if (xwall_warp) ph = __shfl_sync(FULL, ph, src);
    ph_m = ph;
    phl_m = __shfl_up_sync(FULL, ph, 1);
  }
  double tsum_m = 0.0, tfc_m = 0.0;  // corrector: top-face sum / flux of the previous row
  // interior body: cell masses rho*vol of columns j and j-1, previous row
  const double vol = dx * dy;
  double mass_m = 0.0, massl_m = 0.0, mass_c = 0.0, massl_c = 0.0;
  if constexpr (!EDGE) {
    const double* a = row(k0 - 1);
    mass_m = a[LF_R * LFS] * vol;
    massl_m = a[LF_R * LFS - 1] * vol;
  }
  double u1_m = 0.0, v1_m = 0.0, u1r_m = 0.0, v1r_m = 0.0;
  // ring rows k-1, k, k+1 of the iteration, rotated at its end (one slot
  // address per row instead of a modulo per access); slot / phase of row k+1
  const double* Pm = row(k0 - 1);
  const double* Pc = row(k0);
  const double* Pn = row(k0 + 1);
  unsigned wsl = 2u % (unsigned)LSTG, wph = 0u;
  unsigned isl = 0u;  // slot of row k-1, refilled at the end of iteration k
  for (int k = k0; k <= k1; ++k) {
    if constexpr (LBOX == 1) {
      mbar_wait(&bars[wsl], wph);  // row k+1
    } else {
      if ((unsigned)(k + 1 - r_first) % (unsigned)LBOX == 0u) wait_row(k + 1);  // its box
    }
    const double* rm = Pm;
    const double* rc = Pc;
    double ph = 0.0;
    if constexpr (EDGE) {
      if (c.wt && k == c.ny + 1)
        ph = ph_m;  // reflective top: mirror of row ny
      else if (colok)
        ph = predict(rc, Pn);
    } else {
      const double* rn = Pn;
      const double tf = pdv_face_pred(rn[LF_V * LFS], rn[LF_V * LFS + 1], dx, dt);
      ph = pdv_predict_pressure_bt(dv, rc[LF_R * LFS], rc[LF_E * LFS], rc[LF_Q * LFS],
                                   rc[LF_U * LFS], rn[LF_U * LFS], rc[LF_U * LFS + 1],
                                   rn[LF_U * LFS + 1], tfp, tf, dx, dy, c.rvol, dt);
      tfp = tf;
    }
    if (xwall_warp) ph = __shfl_sync(FULL, ph, src);
    const double phl = __shfl_up_sync(FULL, ph, 1);

    // accelerate at node (j,k): cells (j-1,k-1), (j,k-1), (j,k), (j-1,k)
    double u1_c = 0.0, v1_c = 0.0;
    if (colok) {
      const double pp[4] = {phl_m, ph_m, ph, phl};
      const double qv[4] = {rm[LF_Q * LFS - 1], rm[LF_Q * LFS], rc[LF_Q * LFS], rc[LF_Q * LFS - 1]};
      if constexpr (EDGE) {
        const double rr[4] = {rm[LF_R * LFS - 1], rm[LF_R * LFS], rc[LF_R * LFS], rc[LF_R * LFS - 1]};
        accelerate_node(dv, rr, pp, qv, rc[LF_U * LFS], rc[LF_V * LFS], dx, dy, dt, u1_c, v1_c);
      } else {
        // cell masses of row k; those of row k-1 are carried from the last row
        mass_c = rc[LF_R * LFS] * vol;
        massl_c = rc[LF_R * LFS - 1] * vol;
        const double mm[4] = {massl_m, mass_m, mass_c, massl_c};
        accelerate_node_m(dv, mm, pp, qv, rc[LF_U * LFS], rc[LF_V * LFS], dx, dy, dt, u1_c, v1_c);
      }
    }
    const double u1r_c = __shfl_down_sync(FULL, u1_c, 1);
    const double v1r_c = __shfl_down_sync(FULL, v1_c, 1);

    // PdV corrector + flux_calc of cell (j,k-1)
    const int kc = k - 1;
    double tsum_c = 0.0, tfc_c = 0.0;
    if constexpr (!EDGE) {
      // top face of cell row k-1 = bottom face of row k (carried to k+1)
      tsum_c = rc[LF_V * LFS] + rc[LF_V * LFS + 1] + v1_c + v1r_c;
      tfc_c = pdv_face_corr(tsum_c, dx, dt);
    }
    if (kc >= k0 && lane >= 1 && lane <= LW && (!EDGE || j <= c.nx)) {
      const double u0_m = rm[LF_U * LFS], u0r_m = rm[LF_U * LFS + 1];
      const double u0_c = rc[LF_U * LFS], u0r_c = rc[LF_U * LFS + 1];
      const double lsum = u0_m + u0_c + u1_m + u1_c;
      const double rsum = u0r_m + u0r_c + u1r_m + u1r_c;
      double bsum, tsum, bfc, tfc;
      if constexpr (EDGE) {
        const double v0_m = rm[LF_V * LFS], v0r_m = rm[LF_V * LFS + 1];
        const double v0_c = rc[LF_V * LFS], v0r_c = rc[LF_V * LFS + 1];
        bsum = v0_m + v0r_m + v1_m + v1r_m;
        tsum = v0_c + v0r_c + v1_c + v1r_c;
        bfc = pdv_face_corr(bsum, dx, dt);
        tfc = pdv_face_corr(tsum, dx, dt);
      } else {
        bsum = tsum_m; tsum = tsum_c;
        bfc = tfc_m; tfc = tfc_c;
      }
      double ev, dvv;
      pdv_correct_bt(dv, rm[LF_R * LFS], rm[LF_E * LFS], ph_m, rm[LF_Q * LFS], lsum, rsum, bfc, tfc,
                     dx, dy, c.rvol, dt, ev, dvv);
      const int ic = idx(c, j, kc);
      const double cx = 0.25 * dt * dy, cy = 0.25 * dt * dx;
      if (!EDGE || !(ncol || near_wall_row(c, kc))) {
        e1[ic] = ev;
        d1[ic] = dvv;
        fx[ic] = cx * lsum;
        fy[ic] = cy * bsum;
        u1[ic] = u1_m;
        v1[ic] = v1_m;
      } else {
        store_mirrored(c, e1, K_CELL, j, kc, ev);
        store_mirrored(c, d1, K_CELL, j, kc, dvv);
        store_mirrored(c, fx, K_XFACE, j, kc, cx * lsum);
        store_mirrored(c, fy, K_YFACE, j, kc, cy * bsum);
        store_mirrored(c, u1, K_XVEL, j, kc, u1_m);
        store_mirrored(c, v1, K_YVEL, j, kc, v1_m);
      }
      if (EDGE && (j == c.nx || kc == c.ny)) {
        if (j == c.nx) {
          store_field(c, fx, K_XFACE, j + 1, kc, cx * rsum);
          store_field(c, u1, K_XVEL, j + 1, kc, u1r_m);
          store_field(c, v1, K_YVEL, j + 1, kc, v1r_m);
        }
        if (kc == c.ny) {
          store_field(c, fy, K_YFACE, j, kc + 1, cy * tsum);
          store_field(c, u1, K_XVEL, j, kc + 1, u1_c);
          store_field(c, v1, K_YVEL, j, kc + 1, v1_c);
        }
        if (j == c.nx && kc == c.ny) {
          store_field(c, u1, K_XVEL, j + 1, kc + 1, u1r_c);
          store_field(c, v1, K_YVEL, j + 1, kc + 1, v1r_c);
        }
      }
    }
    ph_m = ph; phl_m = phl;
    u1_m = u1_c; v1_m = v1_c; u1r_m = u1r_c; v1r_m = v1r_c;
    tsum_m = tsum_c; tfc_m = tfc_c;
    mass_m = mass_c; massl_m = massl_c;
    // row k-1 is consumed (rows k, k+1 are still read next iteration):
    // refill its slot with row k-1+LSTG
#if CLOVER_TMA_RELEASE_FENCE
    fence_proxy_async();
#endif
    __syncwarp();
    if constexpr (LBOX == 1) {
      if (lane == 0 && k - 1 + LSTG <= r_last) issue_at(isl, k - 1 + LSTG);
      if (++isl == (unsigned)LSTG) isl = 0u;
      Pm = Pc; Pc = Pn;
      if (++wsl == (unsigned)LSTG) { wsl = 0u; wph ^= 1u; }
      Pn = ring + wsl * LSLOT + lane + 1;
    } else {
      // row k-1 ends its box: refill the slot with the box LSTG boxes on
      if ((unsigned)(k - 1 - r_first) % (unsigned)LBOX == (unsigned)(LBOX - 1) && lane == 0 &&
          k + (LSTG - 1) * LBOX <= r_last)
        issue(k + (LSTG - 1) * LBOX);
      Pm = Pc; Pc = Pn;
      Pn = row(k + 2);
    }
  }
  __syncwarp();
  if (lane == 0)
    for (int t = 0; t < LSTG; ++t) mbar_inval(&bars[t]);  // the ring may be reused (fixup)
  __syncwarp();
  return __any_sync(FULL, dv.bad);
}

__device__ __forceinline__ bool lagr_interior(const Chunk& c, int gw, int k0, int k1) {
  const int J0 = 1 + LW * gw;
  return J0 - 2 >= HALO + 2 && J0 + 31 <= c.nx - HALO - 1 && k0 - 1 >= HALO + 2 &&
         k1 + 1 <= c.ny - HALO - 1;
}

template <class D>
__device__ __forceinline__ bool lagr_seg(const Chunk& c, const CUtensorMap* __restrict__ tm,
                                         double* __restrict__ d1, double* __restrict__ e1,
                                         double* __restrict__ u1, double* __restrict__ v1,
                                         double* __restrict__ fx, double* __restrict__ fy,
                                         const StepScalars* __restrict__ s, int gw, int k0, int k1,
                                         int lane, double* ring, unsigned long long* bars) {
  if (lagr_interior(c, gw, k0, k1))
    return lagr_body<D, false>(c, tm, d1, e1, u1, v1, fx, fy, s, gw, k0, k1, lane, ring, bars);
  return lagr_body<D, true>(c, tm, d1, e1, u1, v1, fx, fy, s, gw, k0, k1, lane, ring, bars);
}

__global__ void LB_HEAVY
ks_lagrangian(Chunk c, const __grid_constant__ CUtensorMap tm, double* __restrict__ d1,
              double* __restrict__ e1, double* __restrict__ u1, double* __restrict__ v1,
              double* __restrict__ fx, double* __restrict__ fy, const StepScalars* __restrict__ s,
              FixSlot fix) {
  pdl_trigger();
  pdl_wait();
  __shared__ __align__(128) double ring[SB / 32][LSTG * LSLOT];
  __shared__ __align__(8) unsigned long long bars[SB / 32][LSTG];
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  const int gw = blockIdx.x * (SB / 32) + w;
  int k0, len;
  const int sg = seg_y(c);
  seg_rows_lay(sg, c.lks, c.lnb, c.lch, c.lcf, c.ny, k0, len, c.ltd);
  if (len <= 0) return;  // empty band segment
  const int k1 = min(k0 + len, c.ny + 1);
  if (lagr_seg<DivFast>(c, &tm, d1, e1, u1, v1, fx, fy, s, gw, k0, k1, lane, ring[w], bars[w]))
    fix_push(fix, lane, gw, (unsigned)sg);
}

__global__ void __launch_bounds__(SB)
kf_lagrangian(Chunk c, const __grid_constant__ CUtensorMap tm, double* __restrict__ d1,
              double* __restrict__ e1, double* __restrict__ u1, double* __restrict__ v1,
              double* __restrict__ fx, double* __restrict__ fy, StepScalars* __restrict__ s,
              FixSlot fix, YWalls yw) {
  pdl_trigger();
  pdl_wait();
  if (y_walls_after_fix<1>(c, fix, yw)) return;
  __shared__ __align__(128) double ring[SB / 32][LSTG * LSLOT];
  __shared__ __align__(8) unsigned long long bars[SB / 32][LSTG];
  fix_loop(fix, c.lks, c.lnb, c.lch, c.lcf, c.ltd, c.ny + 1, [&](int gw, int k0, int k1, int lane, int w) {
    // the IEEE redo's flag is the exact PdV volume test (DivIEEE::vol_check)
    if (lagr_seg<DivIEEE>(c, &tm, d1, e1, u1, v1, fx, fy, s, gw, k0, k1, lane, ring[w], bars[w]) &&
        lane == 0)
      atomicCAS(&s->err, 0, -6);  // CLOVER_ERR_NEG_VOLUME
  });
}
// (a register-only Lagrangian variant was measured 3% slower; see git history)

// ================================================================ advec_cell x
// Warp strip: lane l <-> face/cell column j = J0 + l, J0 = 1 + 31*(warp);
// every lane computes the flux of face j, lanes 0..30 update cell j using
// face j+1 from the next lane.  Rows [k0, k0+CKS).
constexpr int CW_X = 31;
constexpr int CKS = CLOVER_CKS;

template <int SWEEP, class D>
__device__ __forceinline__ bool advec_cell_x_body(const Chunk& c, const double* __restrict__ rho, const double* __restrict__ en,
                const double* __restrict__ fx, const double* __restrict__ fy,
                double* __restrict__ rho_out, double* __restrict__ en_out,
                double* __restrict__ mfx,
    int gw, int k0, int k1, int lane) {
  D dv;
  const int J0 = 1 + CW_X * gw;
  if (J0 > c.nx) return false;
  const int j = J0 + lane;
  const double vol = c.dx * c.dy;
  const int P = c.pitch;
  const bool faceok = j <= c.nx + 1;
  const bool ncol = near_wall_col(c, j);
  STREAM_LOOP
  for (int k = k0; k < k1; ++k) {
    const int i = idx(c, j, k);
    double pv = 0.0, pvl = 0.0, F = 0.0, m = 0.0, ef = 0.0, rr = 0.0, ee = 0.0, flo = 0.0, fhi = 0.0;
    if (faceok) {
      flo = fx[i]; fhi = fx[i + 1];
      F = flo;
      pv = (SWEEP == 1) ? vol + (fhi - flo + fy[i + P] - fy[i]) : vol + fhi - flo;
      rr = rho[i]; ee = en[i];
    }
    pvl = __shfl_up_sync(FULL, pv, 1);
    if (faceok) {
      if (lane == 0) {
        const double fl = fx[i - 1];
        pvl = (SWEEP == 1) ? vol + (flo - fl + fy[i - 1 + P] - fy[i - 1]) : vol + flo - fl;
      }
      double ru, rd, rw, eu, ed, ew, pvd;
      if (F > 0.0) {
        ru = rho[i - 2]; rd = rho[i - 1]; rw = rr;
        eu = en[i - 2]; ed = en[i - 1]; ew = ee;
        pvd = pvl;
      } else {
        const int up = min(j + 1, c.nx + 2) - j;
        ru = rho[i + up]; rd = rr; rw = rho[i - 1];
        eu = en[i + up]; ed = ee; ew = en[i - 1];
        pvd = pv;
      }
      cell_face_flux(dv, F, pvd, ru, rd, rw, eu, ed, ew, m, ef);
    }
    const double mh = __shfl_down_sync(FULL, m, 1);
    const double efh = __shfl_down_sync(FULL, ef, 1);
    if (lane < CW_X && j <= c.nx) {
      double ro, eo;
      cell_update(dv, rr, ee, pv, m, mh, ef, efh, flo, fhi, ro, eo);
      const bool near = ncol || near_wall_row(c, k);
      store_at(c, rho_out, K_CELL, j, k, i, near, ro);
      store_at(c, en_out, K_CELL, j, k, i, near, eo);
      store_at(c, mfx, K_XFACE, j, k, i, near, m);
      if (j == c.nx) store_field(c, mfx, K_XFACE, j + 1, k, mh);
    }
  }
  return __any_sync(FULL, dv.bad);
}

template <int SWEEP>
__global__ void LB_ADV
ks_advec_cell_x(Chunk c, const double* __restrict__ rho, const double* __restrict__ en,
                const double* __restrict__ fx, const double* __restrict__ fy,
                double* __restrict__ rho_out, double* __restrict__ en_out,
                double* __restrict__ mfx, FixSlot fix) {
  pdl_trigger();
  pdl_wait();
  const int lane = threadIdx.x & 31;
  const int gw = blockIdx.x * (SB / 32) + (threadIdx.x >> 5);
  const int k0 = seg_y(c) * CKS + 1, k1 = min(k0 + CKS, c.ny + 1);
  if (advec_cell_x_body<SWEEP, DivFast>(c, rho, en, fx, fy, rho_out, en_out, mfx, gw, k0, k1, lane)) {
    fix_push(fix, lane, gw, (unsigned)seg_y(c));
  }
}

template <int SWEEP>
__global__ void __launch_bounds__(SB)
kf_advec_cell_x(Chunk c, const double* __restrict__ rho, const double* __restrict__ en,
                const double* __restrict__ fx, const double* __restrict__ fy,
                double* __restrict__ rho_out, double* __restrict__ en_out,
                double* __restrict__ mfx, FixSlot fix) {
  pdl_trigger();
  pdl_wait();
  fix_loop(fix, CKS, 0x7fffffff, 0, 0, CLOVER_TAIL_DIV, c.ny + 1, [&](int gw, int k0, int k1, int lane, int) {
    advec_cell_x_body<SWEEP, DivIEEE>(c, rho, en, fx, fy, rho_out, en_out, mfx, gw, k0, k1, lane);
  });
}

// ================================================================ advec_cell y
// Column j = block*128 + tid + 1; streams cell rows [k0, k1).  Iteration k
// computes the flux of face k+1 and updates cell k (face k from the previous
// iteration).  Registers hold density/energy of rows k-1..k+2 and the
// pre-sweep volume of rows k, k+1.
constexpr int CKS_Y = CLOVER_CKS_Y;

// EDGE = false: columns and rows k0-2 .. k1+1 at least HALO+2 away from
// every wall and chunk edge (y_interior).
template <int SWEEP, class D, bool EDGE>
__device__ __forceinline__ bool advec_cell_y_body(const Chunk& c, const double* __restrict__ rho, const double* __restrict__ en,
                const double* __restrict__ fx, const double* __restrict__ fy,
                double* __restrict__ rho_out, double* __restrict__ en_out,
                double* __restrict__ mfy,
    int gw, int k0, int k1, int lane, int jlo = 1, int jhi = 0x7fffffff) {
  // columns jlo + 32*gw + lane <= min(jhi, nx) (ks_cell_y_walls also
  // computes the halo columns 0 / nx+1 at x chunk boundaries)
  D dv;
  const int j = gw * 32 + lane + jlo;
  if (!EDGE || j <= min(jhi, c.nx)) {
    const double vol = c.dx * c.dy;
    const int P = c.pitch;
    auto pre_vol = [&](int i) -> double {
      if (SWEEP == 1) return vol + (fy[i + P] - fy[i] + fx[i + 1] - fx[i]);
      return vol + fy[i + P] - fy[i];
    };
    const bool ncol = EDGE && near_wall_col(c, j);
    int i = idx(c, j, k0);
    // rows k0-2 .. k0+1
    double R0 = rho[i - 2 * P], R1 = rho[i - P], R2 = rho[i], R3 = rho[i + P];
    double E0 = en[i - 2 * P], E1 = en[i - P], E2 = en[i], E3 = en[i + P];
    double pvm = pre_vol(i - P), pv0 = pre_vol(i);
    // face k0
    double m0, ef0;
    {
      const double F = fy[i];
      double ru, rd, rw, eu, ed, ew, pvd;
      if (F > 0.0) {
        ru = R0; rd = R1; rw = R2; eu = E0; ed = E1; ew = E2; pvd = pvm;
      } else {
        ru = R3; rd = R2; rw = R1; eu = E3; ed = E2; ew = E1; pvd = pv0;
      }
      cell_face_flux(dv, F, pvd, ru, rd, rw, eu, ed, ew, m0, ef0);
    }
    STREAM_LOOP
    for (int k = k0; k < k1; ++k, i += P) {
      // registers: R1..R3 = rows k-1..k+1; load row k+2
      const double R4 = rho[i + 2 * P], E4 = en[i + 2 * P];
      const double pv1 = pre_vol(i + P);
      // face k+1: up = k (F>0: k-1+1), don = k, dw = k+1 ; else up = k+2, don = k+1, dw = k
      double m1, ef1;
      {
        const double F = fy[i + P];
        double ru, rd, rw, eu, ed, ew, pvd;
        if (F > 0.0) {
          ru = R1; rd = R2; rw = R3; eu = E1; ed = E2; ew = E3; pvd = pv0;
        } else {
          ru = R4; rd = R3; rw = R2; eu = E4; ed = E3; ew = E2; pvd = pv1;
        }
        cell_face_flux(dv, F, pvd, ru, rd, rw, eu, ed, ew, m1, ef1);
      }
      double ro, eo;
      {
        const double flo = fy[i], fhi = fy[i + P];
        cell_update(dv, R2, E2, pv0, m0, m1, ef0, ef1, flo, fhi, ro, eo);
      }
      const bool near = EDGE && (ncol || near_wall_row(c, k));
      store_at(c, rho_out, K_CELL, j, k, i, near, ro);
      store_at(c, en_out, K_CELL, j, k, i, near, eo);
      store_at(c, mfy, K_YFACE, j, k, i, near, m0);
      if (EDGE && k == c.ny) store_field(c, mfy, K_YFACE, j, k + 1, m1);
      R0 = R1; R1 = R2; R2 = R3; R3 = R4;
      E0 = E1; E1 = E2; E2 = E3; E3 = E4;
      pvm = pv0; pv0 = pv1;
      m0 = m1; ef0 = ef1;
    }
  }
  return __any_sync(FULL, dv.bad);
}

// columns j = 32*gw+1 .. 32*gw+32 with reach j-1 .. j+2, rows k0-2 .. k1+1
__device__ __forceinline__ bool y_interior(const Chunk& c, int gw, int k0, int k1) {
  return gw * 32 >= HALO + 2 && gw * 32 + 34 <= c.nx - HALO - 1 && k0 - 2 >= HALO + 2 &&
         k1 + 1 <= c.ny - HALO - 1;
}

template <int SWEEP>
__global__ void LB_ADV
ks_advec_cell_y(Chunk c, const double* __restrict__ rho, const double* __restrict__ en,
                const double* __restrict__ fx, const double* __restrict__ fy,
                double* __restrict__ rho_out, double* __restrict__ en_out,
                double* __restrict__ mfy, FixSlot fix) {
  pdl_trigger();
  pdl_wait();
  const int lane = threadIdx.x & 31;
  const int gw = blockIdx.x * (SB / 32) + (threadIdx.x >> 5);
  const int k0 = seg_y(c) * CKS_Y + 1, k1 = min(k0 + CKS_Y, c.ny + 1);
  if (y_interior(c, gw, k0, k1) ? advec_cell_y_body<SWEEP, DivFast, false>(c, rho, en, fx, fy, rho_out, en_out, mfy, gw, k0, k1, lane)
                                : advec_cell_y_body<SWEEP, DivFast, true>(c, rho, en, fx, fy, rho_out, en_out, mfy, gw, k0, k1, lane)) {
    fix_push(fix, lane, gw, (unsigned)seg_y(c));
  }
}

template <int SWEEP>
__global__ void __launch_bounds__(SB)
kf_advec_cell_y(Chunk c, const double* __restrict__ rho, const double* __restrict__ en,
                const double* __restrict__ fx, const double* __restrict__ fy,
                double* __restrict__ rho_out, double* __restrict__ en_out,
                double* __restrict__ mfy, FixSlot fix) {
  pdl_trigger();
  pdl_wait();
  fix_loop(fix, CKS_Y, 0x7fffffff, 0, 0, CLOVER_TAIL_DIV, c.ny + 1, [&](int gw, int k0, int k1, int lane, int) {
    advec_cell_y_body<SWEEP, DivIEEE, true>(c, rho, en, fx, fy, rho_out, en_out, mfy, gw, k0, k1, lane);
  });
}

// ================================================================ advec_mom x
// Warp strip: lane l <-> node column j = J0 - 2 + l, J0 = 1 + 29*(warp);
// lanes 2..30 update nodes j.  Per node row k: node flux from the mass
// fluxes of faces j, j+1 (rows k-1, k), node masses from cells j-1, j
// (rows k-1, k; column j-1 via shuffle), momentum fluxes for u and v.
constexpr int MW_X = 29;
constexpr int MKS = CLOVER_MKS;

template <int SWEEP, class D>
__device__ __forceinline__ bool advec_mom_x_body(const Chunk& c, const double* __restrict__ rho, const double* __restrict__ mfx,
               const double* __restrict__ fy, const double* __restrict__ uin,
               const double* __restrict__ vin, double* __restrict__ uout,
               double* __restrict__ vout,
    int gw, int k0, int k1, int lane) {
  D dv;
  const int J0 = 1 + MW_X * gw;
  if (J0 > c.nx + 1) return false;
  const int j = J0 - 2 + lane;
  const double vol = c.dx * c.dy;
  const int P = c.pitch;
  const bool nfok = j <= c.nx + 2;   // node flux / node mass columns
  const bool ncol = near_wall_col(c, j);
  auto mass_post = [&](int i) -> double {
    const double pv = (SWEEP == 1) ? vol + fy[i + P] - fy[i] : vol;
    return rho[i] * pv;
  };
  double mA_m = 0.0, mB_m = 0.0, mp_m = 0.0;  // row k-1: Mx(j), Mx(j+1), mass of cell (j,k-1)
  if (nfok) {
    const int i = idx(c, j, k0 - 1);
    mA_m = mfx[i]; mB_m = mfx[i + 1]; mp_m = mass_post(i);
  }
  double mpl_m = __shfl_up_sync(FULL, mp_m, 1);
  STREAM_LOOP
  for (int k = k0; k < k1; ++k) {
    const int i = idx(c, j, k);
    double mA = 0.0, mB = 0.0, mp = 0.0;
    if (nfok) {
      mA = mfx[i]; mB = mfx[i + 1]; mp = mass_post(i);
    }
    const double mpl = __shfl_up_sync(FULL, mp, 1);
    const double nf = 0.25 * (mA_m + mA + mB_m + mB);
    const double post = 0.25 * (mp_m + mp + mpl_m + mpl);
    const double nfl = __shfl_up_sync(FULL, nf, 1);
    const double pre = post - nfl + nf;
    const double prer = __shfl_down_sync(FULL, pre, 1);
    double mu = 0.0, mv = 0.0;
    if (lane >= 1 && lane <= 30 && j <= c.nx + 1) {
      int up, don, dw;
      double nmp;
      if (nf < 0.0) {
        up = 2; don = 1; dw = 0; nmp = prer;
      } else {
        up = -1; don = 0; dw = 1; nmp = pre;
      }
      const double uu[3] = {uin[i + up], uin[i + don], uin[i + dw]};
      const double vv[3] = {vin[i + up], vin[i + don], vin[i + dw]};
      mom_flux2(dv, nf, nmp, uu, vv, c.dx, c.rdx, mu, mv);
    }
    const double mul = __shfl_up_sync(FULL, mu, 1);
    const double mvl = __shfl_up_sync(FULL, mv, 1);
    if (lane >= 2 && lane <= MW_X + 1 && j <= c.nx + 1) {
      const double u = uin[i], v = vin[i];
      double un, vn;
      mom_update(dv, u, v, pre, post, mul, mu, mvl, mv, un, vn);
      const bool near = ncol || near_wall_row(c, k);
      store_at(c, uout, K_XVEL, j, k, i, near, un);
      store_at(c, vout, K_YVEL, j, k, i, near, vn);
    }
    mA_m = mA; mB_m = mB; mp_m = mp; mpl_m = mpl;
  }
  return __any_sync(FULL, dv.bad);
}

template <int SWEEP>
__global__ void LB_ADV
ks_advec_mom_x(Chunk c, const double* __restrict__ rho, const double* __restrict__ mfx,
               const double* __restrict__ fy, const double* __restrict__ uin,
               const double* __restrict__ vin, double* __restrict__ uout,
               double* __restrict__ vout, FixSlot fix) {
  pdl_trigger();
  pdl_wait();
  const int lane = threadIdx.x & 31;
  const int gw = blockIdx.x * (SB / 32) + (threadIdx.x >> 5);
  const int k0 = seg_y(c) * MKS + 1, k1 = min(k0 + MKS, c.ny + 2);
  if (advec_mom_x_body<SWEEP, DivFast>(c, rho, mfx, fy, uin, vin, uout, vout, gw, k0, k1, lane)) {
    fix_push(fix, lane, gw, (unsigned)seg_y(c));
  }
}

template <int SWEEP>
__global__ void __launch_bounds__(SB)
kf_advec_mom_x(Chunk c, const double* __restrict__ rho, const double* __restrict__ mfx,
               const double* __restrict__ fy, const double* __restrict__ uin,
               const double* __restrict__ vin, double* __restrict__ uout,
               double* __restrict__ vout, FixSlot fix) {
  pdl_trigger();
  pdl_wait();
  fix_loop(fix, MKS, 0x7fffffff, 0, 0, CLOVER_TAIL_DIV, c.ny + 2, [&](int gw, int k0, int k1, int lane, int) {
    advec_mom_x_body<SWEEP, DivIEEE>(c, rho, mfx, fy, uin, vin, uout, vout, gw, k0, k1, lane);
  });
}

// ================================================================ fused x sweep
// advec_cell (x) and advec_mom (x) of one sweep in one pass (geometric face
// mirror).  At x walls the halo columns are mirrors of lanes of the same
// warp; at x chunk boundaries they are recomputed from inputs exchanged
// HALO_COLS deep (reach: cells j-3 .. j+3, x-faces depth 3).
// Warp strip: lane l <-> column j = J0 - 2 + l, J0 = 1 + 28*(warp).  At cell
// row r every lane computes the x-face flux of face j and (lanes 0..30) the
// cell update of cell j; lanes on wall halo columns take the mirror image of
// the computed interior value instead (the reference's update_halo after
// advec_cell: density/energy mirror with +, x-face mass flux with -), so
// the mass flux and post-advection density the momentum update reads never
// travel through memory.  Node row r then follows as in ks_advec_mom_x
// (node flux from rows r-1, r; masses of cells j-1, j).  Lanes 2..29 own
// cells and nodes.  Cell rows k0-1 .. k1-1 are computed (the first one
// repeats the previous segment's last row).  Halo rows: at a y wall the
// mirror of the adjacent interior row, at a chunk boundary computed from the
// depth-2 input halos (bitwise what the neighbour computes).
constexpr int XW = 28;
#ifndef CLOVER_XKS
#define CLOVER_XKS 16
#endif
constexpr int XKS = CLOVER_XKS;

// Rows of the inputs stream through a per-warp XSTG-row shared-memory ring,
// one 3D TMA tensor copy per row.  The engine keeps the inputs of each sweep
// as consecutive equally spaced buffers: sweep 1 reads d1 e1 u1 v1 fy fx,
// sweep 2 reads fx d2 e2 u2 v2 (it never reads fy).  Smem column t of a slot
// holds memory column COL0 + J0 - 4 + t (even: 16-B aligned); lane l reads
// its column j = J0 - 2 + l at t = l + 2 and reaches t = l .. l+4.
template <int SWEEP> struct XF;
template <> struct XF<1> { enum { R = 0, E = 1, U = 2, V = 3, FY = 4, FX = 5, NF = 6 }; };
template <> struct XF<2> { enum { FX = 0, R = 1, E = 2, U = 3, V = 4, NF = 5, FY = -1 }; };
constexpr int XRW = 36;
#ifndef CLOVER_XSTG
#define CLOVER_XSTG 4
#endif
constexpr int XSTG = CLOVER_XSTG;
// rows per tensor copy (ring slot), as for visc_dt (VBOX); slot [field][row][column]
#ifndef CLOVER_XBOX
#define CLOVER_XBOX 1
#endif
constexpr int XBOX = CLOVER_XBOX;
constexpr int XFS = XBOX * XRW;  // field stride in a slot (doubles)
template <int SWEEP>
__host__ __device__ constexpr int xslot() { return (XF<SWEEP>::NF * XFS + 15) / 16 * 16; }  // 128-B multiple
static_assert((COL0 + 1 - 4) % 2 == 0 && XW % 2 == 0, "fused x ring box starts on an even column");

// EDGE = false: a warp segment whose columns and rows are all at least
// HALO+2 away from any wall or chunk edge (see x_interior): every lane
// predicate is constant and no mirror logic runs.
template <int SWEEP, class D, bool EDGE>
__device__ __forceinline__ bool advec_x_body(const Chunk& c, const CUtensorMap* __restrict__ tm,
                                             double* __restrict__ rho_out,
                                             double* __restrict__ en_out,
                                             double* __restrict__ uout,
                                             double* __restrict__ vout, int gw, int k0, int k1,
                                             int lane, double* ring, unsigned long long* bars) {
  using F = XF<SWEEP>;
  constexpr int SL = xslot<SWEEP>();
  constexpr unsigned BYTES = F::NF * XFS * 8;
  D dv;
  const int J0 = 1 + XW * gw;
  if (J0 > c.nx + 1) return false;
  const int j = J0 - 2 + lane;
  const double vol = c.dx * c.dy;
  const int nx = c.nx;
  // at an x wall the halo faces / cells are mirrors of lanes of this warp;
  // at an x chunk boundary (no wall) they are computed from the HALO_COLS
  // deep input halos, bitwise what the neighbour computes
  const bool faceok = !EDGE || ((!c.wl || j >= 1) && (!c.wr || j <= nx + 1));  // faces computed here
  const bool cellok = !EDGE || ((!c.wl || j >= 0) && (!c.wr || j <= nx + 2));  // pre_vol inputs exist
  const bool mpok = !EDGE || ((!c.wl || j >= -1) && (!c.wr || j <= nx + 2));   // node-mass columns
  const bool cellup = !EDGE || ((!c.wl || j >= 1) && (!c.wr || j <= nx));      // cell updates
  const bool ncol = EDGE && near_wall_col(c, j);
  const bool own = lane >= 2 && lane < 2 + XW;
  // mirror sources at the x walls (lanes of this warp, see header)
  int src_m = lane, src_r = lane;
  double sgn_m = 1.0;
  if (EDGE) {
    if (c.wl && j <= 0) { src_m = lane + 2 - 2 * j; src_r = lane + 1 - 2 * j; sgn_m = -1.0; }
    if (c.wr && j >= nx + 2) { src_m = lane + 2 * nx + 2 - 2 * j; sgn_m = -1.0; }
    if (c.wr && j >= nx + 1) src_r = lane + 2 * nx + 1 - 2 * j;
    if (src_m < 0 || src_m > 31) src_m = lane;
    if (src_r < 0 || src_r > 31) src_r = lane;
  }
  const bool xwall_warp = EDGE && __any_sync(FULL, src_m != lane || src_r != lane);

  const int r_first = k0 - 1, r_last = k1;  // staged rows (fy of row r+1 is read at row r)
  const int xcol = COL0 + J0 - 4;
  auto slot_of = [&](int r) { return ((unsigned)(r - r_first) / (unsigned)XBOX) % (unsigned)XSTG; };
  auto issue = [&](int r) {
    const unsigned sl = slot_of(r);
    mbar_arrive_expect_tx(&bars[sl], BYTES);
    tma_load_3d(ring + sl * SL, tm, xcol, c.row0 + r, 0, &bars[sl]);
  };
  auto wait_row = [&](int r) {
    const unsigned box = (unsigned)(r - r_first) / (unsigned)XBOX;
    mbar_wait(&bars[box % XSTG], (box / XSTG) & 1u);
  };
  auto row = [&](int r) -> const double* {
    return ring + slot_of(r) * SL + ((unsigned)(r - r_first) % (unsigned)XBOX) * XRW + lane + 2;
  };
  // post-sweep cell volume of the node-mass term
  auto pv_mom = [&](const double* rc, const double* rn) -> double {
    if constexpr (SWEEP == 1) return vol + rn[F::FY * XFS] - rc[F::FY * XFS];
    else return vol;
  };
  if (lane == 0) {
    for (int t = 0; t < XSTG; ++t) mbar_init(&bars[t], 1);
    fence_mbar_init();
    fence_proxy_async();
    for (int r = r_first; r < r_first + XSTG * XBOX && r <= r_last; r += XBOX) issue(r);
  }
  __syncwarp();
  wait_row(r_first);

  double mA_m = 0.0, mp_m = 0.0, mB_m = 0.0, mpl_m = 0.0, ro_m = 0.0;
  // (ring slots by mask: XSTG is a power of two; rotating the row pointers
  // as the Lagrangian and y-sweep bodies do cost 8 registers and 2.7 % on
  // sweep 1 here)
  for (int r = k0 - 1; r < k1; ++r) {
    wait_row(r + 1);
    const bool mir_bot = EDGE && c.wb && r == 0;  // synthesised from row 1 below
    if (!mir_bot) {
      const double* rc = row(r);
      const double* rn = row(r + 1);
      const int i = idx(c, j, r);
      const bool mir_top = EDGE && c.wt && r == c.ny + 1;
      double mA = 0.0, ro = 0.0;
      if (mir_top) {
        // row ny+1 = mirror of row ny (already mirrored along x)
        mA = mA_m; ro = ro_m;
      } else {
        // ---- advec_cell x, row r
        double pv = 0.0, F = 0.0, m = 0.0, ef = 0.0, rr = 0.0, ee = 0.0, flo = 0.0, fhi = 0.0;
        if (cellok) {
          flo = rc[F::FX * XFS]; fhi = rc[F::FX * XFS + 1];
          F = flo;
          if constexpr (SWEEP == 1)
            pv = vol + (fhi - flo + rn[F::FY * XFS] - rc[F::FY * XFS]);
          else
            pv = vol + fhi - flo;
          rr = rc[F::R * XFS]; ee = rc[F::E * XFS];
        }
        if (faceok) {
          // pre_vol of cell j-1 from the ring (the same expression lane j-1
          // evaluates: same bits; cheaper than a 64-bit shuffle plus a
          // divergent lane-0 path)
          double pvl;
          {
            const double fl = rc[F::FX * XFS - 1];
            if constexpr (SWEEP == 1)
              pvl = vol + (flo - fl + rn[F::FY * XFS - 1] - rc[F::FY * XFS - 1]);
            else
              pvl = vol + flo - fl;
          }
          // upwind / donor / downwind columns picked by address (one select
          // per column instead of one per loaded value)
          const bool pos = F > 0.0;
          // (the reading's MIN(j+1, x_max+2) upwind clamp only acts at a wall)
          const double* pu = pos ? rc - 2 : rc + ((EDGE && c.wr) ? min(j + 1, nx + 2) - j : 1);
          const double* pd = pos ? rc - 1 : rc;
          const double* pw = pos ? rc : rc - 1;
          cell_face_flux(dv, F, pos ? pvl : pv, pu[F::R * XFS], pd[F::R * XFS], pw[F::R * XFS],
                         pu[F::E * XFS], pd[F::E * XFS], pw[F::E * XFS], m, ef);
        }
        const double mh = __shfl_down_sync(FULL, m, 1);
        const double efh = __shfl_down_sync(FULL, ef, 1);
        double eo = 0.0;
        if (cellup && lane < 31) {
          cell_update(dv, rr, ee, pv, m, mh, ef, efh, flo, fhi, ro, eo);
          if (own && r >= k0 && (!EDGE || r <= c.ny)) {
            const bool near = EDGE && (ncol || near_wall_row(c, r));
            store_at(c, rho_out, K_CELL, j, r, i, near, ro);
            store_at(c, en_out, K_CELL, j, r, i, near, eo);
          }
        }
        mA = m;
        if (xwall_warp) {
          const double ms = __shfl_sync(FULL, m, src_m);
          const double rs = __shfl_sync(FULL, ro, src_r);
          if (src_m != lane) mA = sgn_m * ms;
          if (src_r != lane) ro = rs;
        }
      }
      const double mB = __shfl_down_sync(FULL, mA, 1);
      double mp = 0.0;
      if (mpok) mp = ro * pv_mom(rc, rn);
      const double mpl = __shfl_up_sync(FULL, mp, 1);
      if (EDGE && c.wb && r == 1) {
        // row 0 = mirror of row 1: same mass fluxes and density, row-0 volumes
        mA_m = mA; mB_m = mB;
        mp_m = mpok ? ro * pv_mom(row(0), rc) : 0.0;
        mpl_m = __shfl_up_sync(FULL, mp_m, 1);
      }
      if (r >= k0) {
        // ---- advec_mom x, node row r
        const double nf = 0.25 * (mA_m + mA + mB_m + mB);
        const double post = 0.25 * (mp_m + mp + mpl_m + mpl);
        const double nfl = __shfl_up_sync(FULL, nf, 1);
        const double pre = post - nfl + nf;
        const double prer = __shfl_down_sync(FULL, pre, 1);
        double mu = 0.0, mv = 0.0;
        if (lane >= 1 && lane <= 29 && (!EDGE || j <= nx + 1)) {
          int up, don, dw;
          double nmp;
          if (nf < 0.0) {
            up = 2; don = 1; dw = 0; nmp = prer;
          } else {
            up = -1; don = 0; dw = 1; nmp = pre;
          }
          const double uu[3] = {rc[F::U * XFS + up], rc[F::U * XFS + don], rc[F::U * XFS + dw]};
          const double vv[3] = {rc[F::V * XFS + up], rc[F::V * XFS + don], rc[F::V * XFS + dw]};
          mom_flux2(dv, nf, nmp, uu, vv, c.dx, c.rdx, mu, mv);
        }
        const double mul = __shfl_up_sync(FULL, mu, 1);
        const double mvl = __shfl_up_sync(FULL, mv, 1);
        if (own && (!EDGE || (j >= 1 && j <= nx + 1))) {
          const double u = rc[F::U * XFS], v = rc[F::V * XFS];
          double un, vn;
          mom_update(dv, u, v, pre, post, mul, mu, mvl, mv, un, vn);
          const bool near = EDGE && (ncol || near_wall_row(c, r));
          store_at(c, uout, K_XVEL, j, r, i, near, un);
          store_at(c, vout, K_YVEL, j, r, i, near, vn);
        }
      }
      mA_m = mA; mB_m = mB; mp_m = mp; mpl_m = mpl; ro_m = ro;
    }
    // row r-1 is consumed (row 0 is read at r = 1): refill its slot
    if (r > r_first) {
#if CLOVER_TMA_RELEASE_FENCE
      fence_proxy_async();
#endif
      __syncwarp();
      if constexpr (XBOX == 1) {
        if (lane == 0 && r - 1 + XSTG <= r_last) issue(r - 1 + XSTG);
      } else {  // row r-1 ends its box: refill the slot with the box XSTG boxes on
        if ((unsigned)(r - 1 - r_first) % (unsigned)XBOX == (unsigned)(XBOX - 1) && lane == 0 &&
            r + (XSTG - 1) * XBOX <= r_last)
          issue(r + (XSTG - 1) * XBOX);
      }
    }
  }
  __syncwarp();
  if (lane == 0)
    for (int t = 0; t < XSTG; ++t) mbar_inval(&bars[t]);  // the ring may be reused (fixup)
  __syncwarp();
  return __any_sync(FULL, dv.bad);
}

// A warp segment is interior when every lane column j = J0-2 .. J0+29 and
// its stencil reach (j-2 .. j+2) lie in [HALO+2, nx-HALO-1] and every row
// r = k0-1 .. k1 in [HALO+2, ny-HALO-1]: no wall mirror, halo row or
// near-wall store can occur.
__device__ __forceinline__ bool x_interior(const Chunk& c, int gw, int k0, int k1) {
  const int J0 = 1 + XW * gw;
  return J0 - 4 >= HALO + 2 && J0 + 31 <= c.nx - HALO - 1 && k0 - 1 >= HALO + 2 &&
         k1 <= c.ny - HALO - 1;
}

template <int SWEEP, class D>
__device__ __forceinline__ bool advec_x_seg(const Chunk& c, const CUtensorMap* __restrict__ tm,
                                            double* __restrict__ rho_out,
                                            double* __restrict__ en_out,
                                            double* __restrict__ uout, double* __restrict__ vout,
                                            int gw, int k0, int k1, int lane, double* ring,
                                            unsigned long long* bars) {
  if (x_interior(c, gw, k0, k1))
    return advec_x_body<SWEEP, D, false>(c, tm, rho_out, en_out, uout, vout, gw, k0, k1, lane,
                                         ring, bars);
  return advec_x_body<SWEEP, D, true>(c, tm, rho_out, en_out, uout, vout, gw, k0, k1, lane, ring,
                                      bars);
}

template <int SWEEP>
__global__ void LB_ADVX
ks_advec_x(Chunk c, const __grid_constant__ CUtensorMap tm, double* __restrict__ rho_out,
           double* __restrict__ en_out, double* __restrict__ uout, double* __restrict__ vout,
           FixSlot fix) {
  pdl_trigger();
  pdl_wait();
  __shared__ __align__(128) double ring[SB / 32][XSTG * xslot<SWEEP>()];
  __shared__ __align__(8) unsigned long long bars[SB / 32][XSTG];
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  const int gw = blockIdx.x * (SB / 32) + w;
  int k0, len;
  const int sg = seg_y(c);
  seg_rows_lay(sg, c.xks, c.xnb, c.xch, c.xcf, c.ny + 1, k0, len, c.xtd);
  if (len <= 0) return;  // empty band segment
  const int k1 = min(k0 + len, c.ny + 2);
  if (advec_x_seg<SWEEP, DivFast>(c, &tm, rho_out, en_out, uout, vout, gw, k0, k1, lane, ring[w],
                                   bars[w]))
    fix_push(fix, lane, gw, (unsigned)sg);
}

template <int SWEEP>
__global__ void __launch_bounds__(SB)
kf_advec_x(Chunk c, const __grid_constant__ CUtensorMap tm, double* __restrict__ rho_out,
           double* __restrict__ en_out, double* __restrict__ uout, double* __restrict__ vout,
           FixSlot fix, YWalls yw) {
  pdl_trigger();
  pdl_wait();
  if constexpr (SWEEP == 1)  // sweep 2 is y
    if (y_walls_after_fix<2>(c, fix, yw)) return;
  __shared__ __align__(128) double ring[SB / 32][XSTG * xslot<SWEEP>()];
  __shared__ __align__(8) unsigned long long bars[SB / 32][XSTG];
  fix_loop(fix, c.xks, c.xnb, c.xch, c.xcf, c.xtd, c.ny + 2, [&](int gw, int k0, int k1, int lane, int w) {
    advec_x_seg<SWEEP, DivIEEE>(c, &tm, rho_out, en_out, uout, vout, gw, k0, k1, lane, ring[w],
                                 bars[w]);
  });
}

// ================================================================ advec_mom y
// Column j = block*128 + tid + 1 (node column), streams node rows [k0, k1).
// Iteration k computes node flux / node masses of row k+1, the momentum
// flux of row k and updates node k.
constexpr int MKS_Y = CLOVER_MKS_Y;

// EDGE = false: see y_interior.
template <int SWEEP, class D, bool EDGE>
__device__ __forceinline__ bool advec_mom_y_body(const Chunk& c, const double* __restrict__ rho, const double* __restrict__ mfy,
               const double* __restrict__ fx, const double* __restrict__ uin,
               const double* __restrict__ vin, double* __restrict__ uout,
               double* __restrict__ vout,
    int gw, int k0, int k1, int lane) {
  D dv;
  const int j = gw * 32 + lane + 1;
  if (!EDGE || j <= c.nx + 1) {
    const double vol = c.dx * c.dy;
    const int P = c.pitch;
    auto mass_post = [&](int i) -> double {  // rho * post_vol of the cell at offset i
      const double pv = (SWEEP == 1) ? vol + fx[i + 1] - fx[i] : vol;
      return rho[i] * pv;
    };
    const bool ncol = EDGE && near_wall_col(c, j);
    // node flux of row r uses My(j-1,r), My(j,r), My(j-1,r+1), My(j,r+1)
    auto node_flux = [&](int i) -> double {
      return 0.25 * (mfy[i - 1] + mfy[i] + mfy[i - 1 + P] + mfy[i + P]);
    };
    // node mass post of row r uses cells (j,r-1), (j,r), (j-1,r-1), (j-1,r)
    auto node_post = [&](double mj_m, double mj, double ml_m, double ml) -> double {
      return 0.25 * (mj_m + mj + ml_m + ml);
    };
    int i = idx(c, j, k0);
    // prologue: rows k0-2 .. k0
    double mpj_a = mass_post(i - 2 * P), mpl_a = mass_post(i - 2 * P - 1);  // row k0-2
    double mpj_b = mass_post(i - P), mpl_b = mass_post(i - P - 1);          // row k0-1
    double mpj_c = mass_post(i), mpl_c = mass_post(i - 1);                  // row k0
    const double nf_m2 = node_flux(i - 2 * P);
    double nf_m = node_flux(i - P);                  // nf(k0-1)
    double nf_0 = node_flux(i);                      // nf(k0)
    const double post_m = node_post(mpj_a, mpj_b, mpl_a, mpl_b);   // nmpost(k0-1)
    double post_0 = node_post(mpj_b, mpj_c, mpl_b, mpl_c);         // nmpost(k0)
    const double pre_m = post_m - nf_m2 + nf_m;                    // nmp(k0-1)
    double pre_0 = post_0 - nf_m + nf_0;                           // nmp(k0)
    double U0 = uin[i - 2 * P], U1 = uin[i - P], U2 = uin[i], U3 = uin[i + P];  // rows k0-2..k0+1
    double V0 = vin[i - 2 * P], V1 = vin[i - P], V2 = vin[i], V3 = vin[i + P];
    double mu_m, mv_m;  // mom flux of row k0-1
    {
      const double nf = nf_m;
      const double nmp = (nf < 0.0) ? pre_0 : pre_m;
      const double uu[3] = {nf < 0.0 ? U3 : U0, nf < 0.0 ? U2 : U1, nf < 0.0 ? U1 : U2};
      const double vv[3] = {nf < 0.0 ? V3 : V0, nf < 0.0 ? V2 : V1, nf < 0.0 ? V1 : V2};
      mom_flux2(dv, nf, nmp, uu, vv, c.dy, c.rdy, mu_m, mv_m);
    }
    STREAM_LOOP
    for (int k = k0; k < k1; ++k, i += P) {
      // registers: U1..U3 = rows k-1..k+1 ; load row k+2
      const double U4 = uin[i + 2 * P], V4 = vin[i + 2 * P];
      const double mpj_d = mass_post(i + P), mpl_d = mass_post(i + P - 1);  // row k+1
      const double nf_1 = node_flux(i + P);                                 // nf(k+1)
      const double post_1 = node_post(mpj_c, mpj_d, mpl_c, mpl_d);          // nmpost(k+1)
      const double pre_1 = post_1 - nf_0 + nf_1;                            // nmp(k+1)
      double mu, mv;
      {
        const double nf = nf_0;
        const double nmp = (nf < 0.0) ? pre_1 : pre_0;
        const double uu[3] = {nf < 0.0 ? U4 : U1, nf < 0.0 ? U3 : U2, nf < 0.0 ? U2 : U3};
        const double vv[3] = {nf < 0.0 ? V4 : V1, nf < 0.0 ? V3 : V2, nf < 0.0 ? V2 : V3};
        mom_flux2(dv, nf, nmp, uu, vv, c.dy, c.rdy, mu, mv);
      }
      double un, vn;
      {
        mom_update(dv, U2, V2, pre_0, post_0, mu_m, mu, mv_m, mv, un, vn);
      }
      const bool near = EDGE && (ncol || near_wall_row(c, k));
      store_at(c, uout, K_XVEL, j, k, i, near, un);
      store_at(c, vout, K_YVEL, j, k, i, near, vn);
      U1 = U2; U2 = U3; U3 = U4;
      V1 = V2; V2 = V3; V3 = V4;
      mpj_c = mpj_d; mpl_c = mpl_d;
      nf_0 = nf_1; post_0 = post_1; pre_0 = pre_1;
      mu_m = mu; mv_m = mv;
    }
  }
  return __any_sync(FULL, dv.bad);
}

template <int SWEEP>
__global__ void LB_MOMY
ks_advec_mom_y(Chunk c, const double* __restrict__ rho, const double* __restrict__ mfy,
               const double* __restrict__ fx, const double* __restrict__ uin,
               const double* __restrict__ vin, double* __restrict__ uout,
               double* __restrict__ vout, FixSlot fix) {
  pdl_trigger();
  pdl_wait();
  const int lane = threadIdx.x & 31;
  const int gw = blockIdx.x * (SB / 32) + (threadIdx.x >> 5);
  const int k0 = seg_y(c) * MKS_Y + 1, k1 = min(k0 + MKS_Y, c.ny + 2);
  if (y_interior(c, gw, k0, k1) ? advec_mom_y_body<SWEEP, DivFast, false>(c, rho, mfy, fx, uin, vin, uout, vout, gw, k0, k1, lane)
                                : advec_mom_y_body<SWEEP, DivFast, true>(c, rho, mfy, fx, uin, vin, uout, vout, gw, k0, k1, lane)) {
    fix_push(fix, lane, gw, (unsigned)seg_y(c));
  }
}

template <int SWEEP>
__global__ void __launch_bounds__(SB)
kf_advec_mom_y(Chunk c, const double* __restrict__ rho, const double* __restrict__ mfy,
               const double* __restrict__ fx, const double* __restrict__ uin,
               const double* __restrict__ vin, double* __restrict__ uout,
               double* __restrict__ vout, FixSlot fix) {
  pdl_trigger();
  pdl_wait();
  fix_loop(fix, MKS_Y, 0x7fffffff, 0, 0, CLOVER_TAIL_DIV, c.ny + 2, [&](int gw, int k0, int k1, int lane, int) {
    advec_mom_y_body<SWEEP, DivIEEE, true>(c, rho, mfy, fx, uin, vin, uout, vout, gw, k0, k1, lane);
  });
}

// ================================================================ fused y sweep
// advec_cell (y) and advec_mom (y) of one sweep in one pass, for chunks with
// reflective walls at both y ends (py == 1) and the geometric face mirror.
// Warp strip: lane l <-> column j = J0 - 1 + l, J0 = 1 + 31*gw; lanes 1..31
// own cells and nodes, lane 0 is a halo lane whose post-sweep density and
// y-face mass flux the node at J0 reads by shuffle.  Rows stream along the
// sweep: iteration s computes the flux of face s+1 and the update of cell s
// (as ks_advec_cell_y), then node flux / masses of row s, the momentum flux of
// node s-1 and the update of node s-2 (as ks_advec_mom_y); the mass flux and
// post-sweep density never travel through memory.  A segment of node rows
// [k0, k1) computes faces [k0-2, k1+1] and cells [k0-2, k1].
// Halo rows at the y walls (faces <= 0 or >= ny+2, cells <= 0 or >= ny+1)
// are the mirrors written by ks_cell_y_walls (advec_cell_y on rows 1..3 and
// ny-1..ny, launched first); halo columns at x walls take the mirror of the
// adjacent lane (density +, y-face mass flux +); at x chunk boundaries they
// are recomputed from the depth-2 input halos.
// Inputs stream through a per-warp ring of YL<SWEEP>::RING rows: sweep 1 reads d1 e1 u1 v1
// fy fx (one 3D tensor copy per row), sweep 2 reads fy and d2 e2 u2 v2 (two).
constexpr int YW = 31;
#ifndef CLOVER_YKS
#define CLOVER_YKS 32
#endif
constexpr int YKS = CLOVER_YKS;
// Ring depth per sweep (rows): sweep 1 (6 fields per row) at 7 rows and a
// register cap of 9 blocks/SM (what its 25 KB of ring per block allows),
// sweep 2 (5 fields) at 7 rows uncapped (10 blocks/SM) -- measured best
// after the ring-pointer rotation (round 2, same box, 3 repeats: step
// 0.8737 -> 0.8693 ms against 6/10 and 8/uncapped; round 1's best were 6
// and 8 rows).  On one-warp blocks sweep 2 takes 6 rows (24 warps/SM by
// shared memory instead of 21; y sweep 2 0.2464 -> 0.2444 ms on the bm
// window, 0.328 -> 0.320 on active flow: profiles/r2_yring2_ab.jsonl).
#ifndef CLOVER_YRING1
#define CLOVER_YRING1 7
#endif
#ifndef CLOVER_YRING2
#define CLOVER_YRING2 6
#endif
#ifndef CLOVER_YMINB1  // (18 one-warp blocks: 94 registers; uncapped it takes 106, 2 % slower)
#define CLOVER_YMINB1 (9 * 64 / CLOVER_SB)
#endif
#ifndef CLOVER_L2HINT  // y sweep: L2 policy for the ring rows shared with the segment below
#define CLOVER_L2HINT 0
#endif
#ifndef CLOVER_YWALLS_FOLD  // y-wall bands carried by the preceding fixup launch
#define CLOVER_YWALLS_FOLD 1
#endif
constexpr int YRW = 36;
template <int SWEEP> struct YL;
template <> struct YL<1> {  // tensor d1 e1 u1 v1 fy fx
  static constexpr int RING = CLOVER_YRING1, MINB = CLOVER_YMINB1;
  enum { R = 0, E = YRW, U = 2 * YRW, V = 3 * YRW, FY = 4 * YRW, FX = 5 * YRW, B = 0,
         SLOT = (6 * YRW + 15) / 16 * 16 };
  static constexpr unsigned BYTES = 6 * YRW * 8;
  static constexpr bool TWO = false;
};
// CLOVER_Y2ONE: sweep 2 reads fy fx d2 e2 u2 v2 as one tensor copy per row
// (fx is not used: one copy instead of two for 20 % more bytes)
#ifndef CLOVER_Y2ONE
#define CLOVER_Y2ONE 0
#endif
#if CLOVER_Y2ONE
template <> struct YL<2> {  // tensor fy fx d2 e2 u2 v2
  static constexpr int RING = CLOVER_YRING2, MINB = 0;
  enum { FY = 0, FX = YRW, B = 0, R = 2 * YRW, E = 3 * YRW, U = 4 * YRW, V = 5 * YRW,
         SLOT = (6 * YRW + 15) / 16 * 16 };
  static constexpr unsigned BYTES = 6 * YRW * 8;
  static constexpr bool TWO = false;
};
#else
template <> struct YL<2> {  // tensors fy | d2 e2 u2 v2
  static constexpr int RING = CLOVER_YRING2, MINB = 0;  // 0: no cap
  enum { FY = 0, B = (YRW + 15) / 16 * 16, R = B, E = B + YRW, U = B + 2 * YRW, V = B + 3 * YRW,
         FX = -1, SLOT = (B + 4 * YRW + 15) / 16 * 16 };
  static constexpr unsigned BYTES = 5 * YRW * 8;
  static constexpr bool TWO = true;
};
#endif

template <int SWEEP, class D, bool EDGE>
__device__ __forceinline__ bool advec_y_body(const Chunk& c, const CUtensorMap* __restrict__ ta,
                                             const CUtensorMap* __restrict__ tb,
                                             double* __restrict__ rho_out,
                                             double* __restrict__ en_out,
                                             const double* __restrict__ mfy,
                                             double* __restrict__ uout,
                                             double* __restrict__ vout, int gw, int k0, int k1,
                                             int lane, double* ring, unsigned long long* bars) {
  using L = YL<SWEEP>;
  D dv;
  const int J0 = 1 + YW * gw;
  if (J0 > c.nx + 1) return false;
  const int j = J0 - 1 + lane;
  const int nx = c.nx, ny = c.ny;
  const double vol = c.dx * c.dy;
  // halo columns: mirror at an x wall, recomputed at a chunk boundary
  int src = lane;
  if (EDGE && c.wl && j == 0) src = lane + 1;
  if (EDGE && c.wr && j == nx + 1) src = lane - 1;
  const bool xwall_warp = EDGE && __any_sync(FULL, src != lane);
  const bool comp = !EDGE || (j >= 0 && j <= nx + 1 && src == lane);  // computes its cells/faces
  const bool own_cell = lane >= 1 && (!EDGE || j <= nx);
  const bool own_node = lane >= 1 && (!EDGE || j <= nx + 1);
  const bool ncol = EDGE && near_wall_col(c, j);

  const int r_first = k0 - 4, r_last = k1 + 2;
  const int x0 = COL0 + J0 - 2;
  const int xcol = x0 & ~1;           // 16-B aligned box start
  const int t0 = 1 + (x0 & 1);        // smem column of lane 0
#if CLOVER_L2HINT
  // rows r_first..k0+2 are read again by the segment below at its end, tens
  // of microseconds later: keep them in L2
  const unsigned long long pol_keep = l2_policy_evict_last();
#if CLOVER_L2HINT > 1
  const unsigned long long pol_once = l2_policy_evict_first();
#endif
#endif
  auto issue_at = [&](unsigned sl, int r) {  // row r into slot sl
    double* d = ring + sl * L::SLOT;
    mbar_arrive_expect_tx(&bars[sl], L::BYTES);
#if CLOVER_L2HINT
    if (r <= k0 + 2) {
      tma_load_3d_hint(d, ta, xcol, c.row0 + r, 0, &bars[sl], pol_keep);
      if constexpr (SWEEP == 2 && L::TWO) tma_load_3d_hint(d + L::B, tb, xcol, c.row0 + r, 0, &bars[sl], pol_keep);
      return;
    }
#if CLOVER_L2HINT > 1
    tma_load_3d_hint(d, ta, xcol, c.row0 + r, 0, &bars[sl], pol_once);
    if constexpr (SWEEP == 2 && L::TWO) tma_load_3d_hint(d + L::B, tb, xcol, c.row0 + r, 0, &bars[sl], pol_once);
    return;
#endif
#endif
    tma_load_3d(d, ta, xcol, c.row0 + r, 0, &bars[sl]);
    if constexpr (SWEEP == 2 && L::TWO) tma_load_3d(d + L::B, tb, xcol, c.row0 + r, 0, &bars[sl]);
  };
  auto issue = [&](int r) { issue_at((unsigned)(r - r_first) % (unsigned)L::RING, r); };
  auto row = [&](int r) -> const double* {
    return ring + ((unsigned)(r - r_first) % (unsigned)L::RING) * L::SLOT + lane + t0;
  };
  auto wait_row = [&](int r) {
    const unsigned rel = (unsigned)(r - r_first);
    mbar_wait(&bars[rel % L::RING], (rel / L::RING) & 1u);
  };
  if (lane == 0) {
    for (int t = 0; t < L::RING; ++t) mbar_init(&bars[t], 1);
    fence_mbar_init();
    fence_proxy_async();
    for (int r = r_first; r < r_first + L::RING && r <= r_last; ++r) issue(r);
  }
  __syncwarp();

  // advec_cell pre-sweep volume of a cell row (q) given the next row (qn)
  auto pre_vol_p = [&](const double* q, const double* qn) -> double {
    if constexpr (SWEEP == 1) return vol + (qn[L::FY] - q[L::FY] + q[L::FX + 1] - q[L::FX]);
    else return vol + qn[L::FY] - q[L::FY];
  };
  auto pre_vol = [&](int r) -> double { return pre_vol_p(row(r), row(r + 1)); };
  auto pv_mom_p = [&](const double* q) -> double {  // advec_mom post-sweep volume
    if constexpr (SWEEP == 1) return vol + q[L::FX + 1] - q[L::FX];
    else return vol;
  };
  // at a y wall the faces / cells beyond it are the mirrors ks_cell_y_walls
  // wrote; at a y chunk boundary they are recomputed from the depth-4 input
  // halos (the neighbour computes the same rows from the same inputs: same
  // bits), so no exchange is needed between advec_cell and advec_mom
  auto face_computed = [&](int f) {
    return !EDGE || ((!c.wb || f >= 1) && (!c.wt || f <= ny + 1));
  };
  auto cell_computed = [&](int r) { return !EDGE || ((!c.wb || r >= 1) && (!c.wt || r <= ny)); };
  // flux of face f (between cells f-1 and f) from the ring rows f-2 .. f+1;
  // pvlo = pre_vol(f-1), pvhi = pre_vol(f)
  auto face_flux_p = [&](const double* r2, const double* r1, const double* r0, const double* rp,
                         double pvlo, double pvhi, double& m, double& ef) {
    const double F = r0[L::FY];
    // upwind / donor / downwind rows picked by address (one select per row
    // instead of one per loaded value)
    const bool pos = F > 0.0;
    const double* pu = pos ? r2 : rp;
    const double* pd = pos ? r1 : r0;
    const double* pw = pos ? r0 : r1;
    cell_face_flux(dv, F, pos ? pvlo : pvhi, pu[L::R], pd[L::R], pw[L::R], pu[L::E], pd[L::E],
                   pw[L::E], m, ef);
  };
  auto face_flux = [&](int f, double pvlo, double pvhi, double& m, double& ef) {
    face_flux_p(row(f - 2), row(f - 1), row(f), row(f + 1), pvlo, pvhi, m, ef);
  };

  // ---- prologue: face k0-2
  for (int r = r_first; r <= k0 - 1; ++r) wait_row(r);
  double m_s = 0.0, ef_s = 0.0, pv_s = 0.0;
  {
    const int f = k0 - 2;
    if (face_computed(f)) {
      pv_s = pre_vol(f);
      if (comp) face_flux(f, pre_vol(f - 1), pv_s, m_s, ef_s);
    } else {
      m_s = mfy[idx(c, j, f)];
    }
    if (xwall_warp) {
      const double ms = __shfl_sync(FULL, m_s, src);
      if (src != lane) m_s = ms;
    }
  }
  double myl_s = __shfl_up_sync(FULL, m_s, 1);
  double mp_p = 0.0, mpl_p = 0.0, nf_p = 0.0, pre_p = 0.0, post_p = 0.0;
  double mu_b = 0.0, mv_b = 0.0;  // momentum flux of node s-2
  // ring rows s-2 .. s+2 of the iteration, rotated at its end (one slot
  // address per row instead of one per access); slot / phase of row s+2
  // for its mbarrier wait (rows k0-4 .. k0 are slots 0 .. 4 at s = k0-2)
  static_assert(L::RING >= 5, "the y sweep reads rows s-2 .. s+2");
  const double* Rm2 = row(k0 - 4);
  const double* Rm1 = row(k0 - 3);
  const double* R0 = row(k0 - 2);
  const double* Rp1 = row(k0 - 1);
  const double* Rp2 = row(k0);
  unsigned wsl = 4u % (unsigned)L::RING, wph = 0u;
  unsigned isl = 0u;  // slot of row s-2, refilled at the end of iteration s

#ifdef CLOVER_YUNROLL
  _Pragma(CLOVER_STR(unroll CLOVER_YUNROLL))
#endif
  for (int s = k0 - 2; s <= k1; ++s) {
    if (s + 2 <= r_last) mbar_wait(&bars[wsl], wph);
    {
      // ---- advec_cell y: face s+1, cell s
      double m1 = 0.0, ef1 = 0.0, pv1 = 0.0, ro = 0.0;
      if (face_computed(s + 1)) {
        pv1 = pre_vol_p(Rp1, Rp2);
        if (comp) face_flux_p(Rm1, R0, Rp1, Rp2, pv_s, pv1, m1, ef1);
      } else {
        m1 = mfy[idx(c, j, s + 1)];
      }
      if (cell_computed(s)) {
        if (comp) {
          double eo;
          cell_update(dv, R0[L::R], R0[L::E], pv_s, m_s, m1, ef_s, ef1, R0[L::FY], Rp1[L::FY],
                      ro, eo);
          if (own_cell && s >= k0 && s < k1) {
            const int i = idx(c, j, s);
            const bool near = EDGE && (ncol || near_wall_row(c, s));
            store_at(c, rho_out, K_CELL, j, s, i, near, ro);
            store_at(c, en_out, K_CELL, j, s, i, near, eo);
          }
        }
      } else {
        ro = rho_out[idx(c, j, s)];
      }
      if (xwall_warp) {
        const double ms = __shfl_sync(FULL, m1, src);
        const double rs = __shfl_sync(FULL, ro, src);
        if (src != lane) { m1 = ms; ro = rs; }
      }
      // ---- advec_mom y: node flux / masses of row s
      const double mp = ro * pv_mom_p(R0);
      const double mpl = __shfl_up_sync(FULL, mp, 1);
      const double myl1 = __shfl_up_sync(FULL, m1, 1);
      const double nf = 0.25 * (myl_s + m_s + myl1 + m1);   // My(j-1,s) My(j,s) My(j-1,s+1) My(j,s+1)
      const double post = 0.25 * (mp_p + mp + mpl_p + mpl);  // cells (j,s-1) (j,s) (j-1,s-1) (j-1,s)
      const double pre = post - nf_p + nf;
      // momentum flux of node s-1, then the update of node s-1 (fluxes of
      // nodes s-2 and s-1; node masses of row s-1)
      if (s >= k0 && own_node) {
        const double nfn = nf_p;
        const double nmp = (nfn < 0.0) ? pre : pre_p;
        const double* qm1 = Rm1;
        const double* q0 = R0;
        const bool neg = nfn < 0.0;
        const double* pa = neg ? Rp1 : Rm2;  // upwind
        const double* pb = neg ? q0 : qm1;                 // donor
        const double* pc = neg ? qm1 : q0;                 // downwind
        const double uu[3] = {pa[L::U], pb[L::U], pc[L::U]};
        const double vv[3] = {pa[L::V], pb[L::V], pc[L::V]};
        double mu_c, mv_c;
        mom_flux2(dv, nfn, nmp, uu, vv, c.dy, c.rdy, mu_c, mv_c);
        if (s >= k0 + 1) {
          const int kn = s - 1;
          double un, vn;
          mom_update(dv, qm1[L::U], qm1[L::V], pre_p, post_p, mu_b, mu_c, mv_b, mv_c, un, vn);
          const int i = idx(c, j, kn);
          const bool near = EDGE && (ncol || near_wall_row(c, kn));
          store_at(c, uout, K_XVEL, j, kn, i, near, un);
          store_at(c, vout, K_YVEL, j, kn, i, near, vn);
        }
        mu_b = mu_c; mv_b = mv_c;
      }
      m_s = m1; ef_s = ef1; pv_s = pv1; myl_s = myl1;
      mp_p = mp; mpl_p = mpl; nf_p = nf;
      pre_p = pre; post_p = post;
    }
    // row s-2 is consumed: refill its slot
    if (s - 2 >= r_first) {
#if CLOVER_TMA_RELEASE_FENCE
      fence_proxy_async();
#endif
      __syncwarp();
      if (lane == 0 && s - 2 + L::RING <= r_last) issue_at(isl, s - 2 + L::RING);
    }
    if (++isl == (unsigned)L::RING) isl = 0u;
    Rm2 = Rm1; Rm1 = R0; R0 = Rp1; Rp1 = Rp2;
    if (++wsl == (unsigned)L::RING) { wsl = 0u; wph ^= 1u; }
    Rp2 = ring + wsl * L::SLOT + lane + t0;
  }
  __syncwarp();
  if (lane == 0)
    for (int t = 0; t < L::RING; ++t) mbar_inval(&bars[t]);  // the ring may be reused (fixup)
  __syncwarp();
  return __any_sync(FULL, dv.bad);
}

// interior: columns J0-1 .. J0+31 and rows k0-4 .. k1+2 at least HALO+2 from
// every edge (no halo column, loaded halo row or near-wall store)
__device__ __forceinline__ bool y_fused_interior(const Chunk& c, int gw, int k0, int k1) {
  const int J0 = 1 + YW * gw;
  return J0 - 1 >= HALO + 2 && J0 + 31 <= c.nx - HALO - 1 && k0 - 4 >= HALO + 2 &&
         k1 + 2 <= c.ny - HALO - 1;
}

template <int SWEEP, class D>
__device__ __forceinline__ bool advec_y_seg(const Chunk& c, const CUtensorMap* ta,
                                            const CUtensorMap* tb, double* rho_out, double* en_out,
                                            const double* mfy, double* uout, double* vout, int gw,
                                            int k0, int k1, int lane, double* ring,
                                            unsigned long long* bars) {
  if (y_fused_interior(c, gw, k0, k1))
    return advec_y_body<SWEEP, D, false>(c, ta, tb, rho_out, en_out, mfy, uout, vout, gw, k0, k1,
                                         lane, ring, bars);
  return advec_y_body<SWEEP, D, true>(c, ta, tb, rho_out, en_out, mfy, uout, vout, gw, k0, k1,
                                      lane, ring, bars);
}

template <int SWEEP>
__global__ void __launch_bounds__(SB, YL<SWEEP>::MINB)
ks_advec_y(Chunk c, const __grid_constant__ CUtensorMap ta, const __grid_constant__ CUtensorMap tb,
           double* __restrict__ rho_out, double* __restrict__ en_out, const double* __restrict__ mfy,
           double* __restrict__ uout, double* __restrict__ vout, FixSlot fix) {
  pdl_trigger();
  pdl_wait();
  __shared__ __align__(128) double ring[SB / 32][YL<SWEEP>::RING * YL<SWEEP>::SLOT];
  __shared__ __align__(8) unsigned long long bars[SB / 32][YL<SWEEP>::RING];
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  const int gw = blockIdx.x * (SB / 32) + w;
  int k0, len;
  const int sg = seg_y(c);
  seg_rows_lay(sg, c.yks, c.ynb, c.ych, c.ycf, c.ny + 1, k0, len, c.ytd);
  if (len <= 0) return;  // empty band segment
  const int k1 = min(k0 + len, c.ny + 2);
  if (advec_y_seg<SWEEP, DivFast>(c, &ta, &tb, rho_out, en_out, mfy, uout, vout, gw, k0, k1, lane,
                                  ring[w], bars[w]))
    fix_push(fix, lane, gw, (unsigned)sg);
}

template <int SWEEP>
__global__ void __launch_bounds__(SB)
kf_advec_y(Chunk c, const __grid_constant__ CUtensorMap ta, const __grid_constant__ CUtensorMap tb,
           double* __restrict__ rho_out, double* __restrict__ en_out, const double* __restrict__ mfy,
           double* __restrict__ uout, double* __restrict__ vout, FixSlot fix) {
  pdl_trigger();
  pdl_wait();
  __shared__ __align__(128) double ring[SB / 32][YL<SWEEP>::RING * YL<SWEEP>::SLOT];
  __shared__ __align__(8) unsigned long long bars[SB / 32][YL<SWEEP>::RING];
  fix_loop(fix, c.yks, c.ynb, c.ych, c.ycf, c.ytd, c.ny + 2, [&](int gw, int k0, int k1, int lane, int w) {
    advec_y_seg<SWEEP, DivIEEE>(c, &ta, &tb, rho_out, en_out, mfy, uout, vout, gw, k0, k1, lane,
                                ring[w], bars[w]);
  });
}

// ================================================================ batched launches
// Several chunks of one process in one launch (blockIdx.z = chunk): the
// streaming kernels and their IEEE fixups above, with each chunk's view,
// tensor maps, outputs and fix list taken from one __grid_constant__ array.
// The grid is the largest chunk's; blocks beyond a chunk's strips or row
// segments return at once.  Forward segment order only (Chunk.rev = 0).
// (One chunk per GPU keeps the single-chunk kernels; this removes the
// per-chunk launches and tails when a process owns several chunks.)
constexpr int MAX_BATCH = 16;
template <class A> struct KBatch { A a[MAX_BATCH]; };
struct VArgs { Chunk c; CUtensorMap tm; double* q; FixSlot fix; };
struct LArgs { Chunk c; CUtensorMap tm; double *d1, *e1, *u1, *v1, *fx, *fy; FixSlot fix; };
struct XArgs { Chunk c; CUtensorMap tm; double *rho, *en, *u, *v; FixSlot fix; };
struct YArgs {
  Chunk c; CUtensorMap ta, tb; double *rho, *en; const double* mfy; double *u, *v; FixSlot fix;
};

__global__ void LB_VISC
ks_visc_dt_b(const __grid_constant__ KBatch<VArgs> b, StepScalars* __restrict__ s, DtParams prm) {
  pdl_trigger();
  pdl_wait();
  const VArgs& a = b.a[blockIdx.z];
  const Chunk& c = a.c;
  if ((int)blockIdx.y >= seg_count_lay(c.vks, c.vnb, c.vch, c.vcf, c.ny, c.vtd)) return;
  __shared__ __align__(128) double ring[SBV / 32][VSTG * VSLOT];
  __shared__ __align__(8) unsigned long long bars[SBV / 32][VSTG];
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const int gw = blockIdx.x * (SBV / 32) + warp;
  double dtw = G_BIG;
  int k0, len;
  const int sg = (int)blockIdx.y;
  seg_rows_lay(sg, c.vks, c.vnb, c.vch, c.vcf, c.ny, k0, len, c.vtd);
  if (len <= 0) return;
  int k1 = min(k0 + len, c.ny + 1);
  visc_ring_rows(c, k0, k1);
  if (gw * 32 < c.nx) {
    if (visc_seg<DivFast>(c, &a.tm, a.q, prm, gw, k0, k1, lane, ring[warp], bars[warp], dtw)) {
      fix_push(a.fix, lane, gw, (unsigned)sg);
      dtw = G_BIG;
    }
  }
  __shared__ double wmin[SBV / 32];
  if (lane == 0) wmin[warp] = dtw;
  __syncthreads();
  if (threadIdx.x == 0) {
    double m = wmin[0];
    for (int w = 1; w < SBV / 32; ++w) m = fmin(m, wmin[w]);
    dt_slot_min(s, m);
  }
}
__global__ void __launch_bounds__(SBV)
kf_visc_dt_b(const __grid_constant__ KBatch<VArgs> b, StepScalars* __restrict__ s, DtParams prm) {
  pdl_trigger();
  pdl_wait();
  const VArgs& a = b.a[blockIdx.z];
  const Chunk& c = a.c;
  __shared__ __align__(128) double ring[SBV / 32][VSTG * VSLOT];
  __shared__ __align__(8) unsigned long long bars[SBV / 32][VSTG];
  fix_loop<SBV>(a.fix, c.vks, c.vnb, c.vch, c.vcf, c.vtd, c.ny + 1, [&](int gw, int k0, int k1, int lane, int w) {
    double dtw;
    visc_ring_rows(c, k0, k1);
    visc_seg<DivIEEE>(c, &a.tm, a.q, prm, gw, k0, k1, lane, ring[w], bars[w], dtw);
    if (lane == 0) dt_slot_min(s, dtw);
  });
}

__global__ void LB_HEAVY
ks_lagrangian_b(const __grid_constant__ KBatch<LArgs> b, const StepScalars* __restrict__ s) {
  pdl_trigger();
  pdl_wait();
  const LArgs& a = b.a[blockIdx.z];
  const Chunk& c = a.c;
  if ((int)blockIdx.y >= seg_count_lay(c.lks, c.lnb, c.lch, c.lcf, c.ny, c.ltd)) return;
  __shared__ __align__(128) double ring[SB / 32][LSTG * LSLOT];
  __shared__ __align__(8) unsigned long long bars[SB / 32][LSTG];
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  const int gw = blockIdx.x * (SB / 32) + w;
  int k0, len;
  const int sg = (int)blockIdx.y;
  seg_rows_lay(sg, c.lks, c.lnb, c.lch, c.lcf, c.ny, k0, len, c.ltd);
  if (len <= 0) return;
  const int k1 = min(k0 + len, c.ny + 1);
  if (lagr_seg<DivFast>(c, &a.tm, a.d1, a.e1, a.u1, a.v1, a.fx, a.fy, s, gw, k0, k1, lane, ring[w],
                        bars[w]))
    fix_push(a.fix, lane, gw, (unsigned)sg);
}
__global__ void __launch_bounds__(SB)
kf_lagrangian_b(const __grid_constant__ KBatch<LArgs> b, StepScalars* __restrict__ s) {
  pdl_trigger();
  pdl_wait();
  const LArgs& a = b.a[blockIdx.z];
  const Chunk& c = a.c;
  __shared__ __align__(128) double ring[SB / 32][LSTG * LSLOT];
  __shared__ __align__(8) unsigned long long bars[SB / 32][LSTG];
  fix_loop(a.fix, c.lks, c.lnb, c.lch, c.lcf, c.ltd, c.ny + 1, [&](int gw, int k0, int k1, int lane, int w) {
    if (lagr_seg<DivIEEE>(c, &a.tm, a.d1, a.e1, a.u1, a.v1, a.fx, a.fy, s, gw, k0, k1, lane,
                          ring[w], bars[w]) &&
        lane == 0)
      atomicCAS(&s->err, 0, -6);  // CLOVER_ERR_NEG_VOLUME
  });
}

template <int SWEEP>
__global__ void LB_ADVX ks_advec_x_b(const __grid_constant__ KBatch<XArgs> b) {
  pdl_trigger();
  pdl_wait();
  const XArgs& a = b.a[blockIdx.z];
  const Chunk& c = a.c;
  if ((int)blockIdx.y >= seg_count_lay(c.xks, c.xnb, c.xch, c.xcf, c.ny + 1, c.xtd)) return;
  __shared__ __align__(128) double ring[SB / 32][XSTG * xslot<SWEEP>()];
  __shared__ __align__(8) unsigned long long bars[SB / 32][XSTG];
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  const int gw = blockIdx.x * (SB / 32) + w;
  int k0, len;
  const int sg = (int)blockIdx.y;
  seg_rows_lay(sg, c.xks, c.xnb, c.xch, c.xcf, c.ny + 1, k0, len, c.xtd);
  if (len <= 0) return;
  const int k1 = min(k0 + len, c.ny + 2);
  if (advec_x_seg<SWEEP, DivFast>(c, &a.tm, a.rho, a.en, a.u, a.v, gw, k0, k1, lane, ring[w],
                                   bars[w]))
    fix_push(a.fix, lane, gw, (unsigned)sg);
}
template <int SWEEP>
__global__ void __launch_bounds__(SB) kf_advec_x_b(const __grid_constant__ KBatch<XArgs> b) {
  pdl_trigger();
  pdl_wait();
  const XArgs& a = b.a[blockIdx.z];
  const Chunk& c = a.c;
  __shared__ __align__(128) double ring[SB / 32][XSTG * xslot<SWEEP>()];
  __shared__ __align__(8) unsigned long long bars[SB / 32][XSTG];
  fix_loop(a.fix, c.xks, c.xnb, c.xch, c.xcf, c.xtd, c.ny + 2, [&](int gw, int k0, int k1, int lane, int w) {
    advec_x_seg<SWEEP, DivIEEE>(c, &a.tm, a.rho, a.en, a.u, a.v, gw, k0, k1, lane, ring[w],
                                 bars[w]);
  });
}

template <int SWEEP>
__global__ void __launch_bounds__(SB, YL<SWEEP>::MINB)
ks_advec_y_b(const __grid_constant__ KBatch<YArgs> b) {
  pdl_trigger();
  pdl_wait();
  const YArgs& a = b.a[blockIdx.z];
  const Chunk& c = a.c;
  if ((int)blockIdx.y >= seg_count_lay(c.yks, c.ynb, c.ych, c.ycf, c.ny + 1, c.ytd)) return;
  __shared__ __align__(128) double ring[SB / 32][YL<SWEEP>::RING * YL<SWEEP>::SLOT];
  __shared__ __align__(8) unsigned long long bars[SB / 32][YL<SWEEP>::RING];
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  const int gw = blockIdx.x * (SB / 32) + w;
  int k0, len;
  const int sg = (int)blockIdx.y;
  seg_rows_lay(sg, c.yks, c.ynb, c.ych, c.ycf, c.ny + 1, k0, len, c.ytd);
  if (len <= 0) return;
  const int k1 = min(k0 + len, c.ny + 2);
  if (advec_y_seg<SWEEP, DivFast>(c, &a.ta, &a.tb, a.rho, a.en, a.mfy, a.u, a.v, gw, k0, k1, lane,
                                  ring[w], bars[w]))
    fix_push(a.fix, lane, gw, (unsigned)sg);
}
template <int SWEEP>
__global__ void __launch_bounds__(SB) kf_advec_y_b(const __grid_constant__ KBatch<YArgs> b) {
  pdl_trigger();
  pdl_wait();
  const YArgs& a = b.a[blockIdx.z];
  const Chunk& c = a.c;
  __shared__ __align__(128) double ring[SB / 32][YL<SWEEP>::RING * YL<SWEEP>::SLOT];
  __shared__ __align__(8) unsigned long long bars[SB / 32][YL<SWEEP>::RING];
  fix_loop(a.fix, c.yks, c.ynb, c.ych, c.ycf, c.ytd, c.ny + 2, [&](int gw, int k0, int k1, int lane, int w) {
    advec_y_seg<SWEEP, DivIEEE>(c, &a.ta, &a.tb, a.rho, a.en, a.mfy, a.u, a.v, gw, k0, k1, lane,
                                ring[w], bars[w]);
  });
}

// the y-wall bands as their own launch (several chunks or ranks; see YWalls)
template <int SWEEP>
__global__ void __launch_bounds__(SB)
ks_cell_y_walls(Chunk c, YWalls y) {
  pdl_trigger();
  pdl_wait();
  y_walls_block<SWEEP>(c, y, blockIdx.x, blockIdx.y);
}

}  // namespace clover
