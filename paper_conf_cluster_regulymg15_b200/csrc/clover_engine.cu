// clover_engine.cu -- step engine and C ABI (include/clover.h) of the
// B200-native CloverLeaf 2D timestep.
//
// Owns: the chunk decomposition (sec. II.B: up-front
// partitioning + halo exchanges), the per-step kernel schedule (SURVEY.md
// 3(ii) hydro order, fused as in DESIGN.md "Kernels"), the device-resident
// dt reduction, halo exchange phases (device-to-device copies between local
// chunks; NCCL send/recv between ranks), CUDA-graph capture of the step,
// and the deterministic field_summary.
#include <cuda_runtime.h>

#include <algorithm>
#include <cmath>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <string>
#include <utility>
#include <vector>

#include "clover.h"
#include "clover_aux.cuh"
#include "clover_common.cuh"
#include "clover_kernels.cuh"
#include "clover_stream.cuh"

#ifdef CLOVER_WITH_NCCL
#include <nccl.h>
#include <nccl_device.h>  // symmetric windows + LSA barrier (device-initiated halo stores)
#endif

using namespace clover;

namespace {

thread_local std::string g_last_error;

int fail(int code, const std::string& msg) {
  g_last_error = msg;
  return code;
}

#define CK(call)                                                                   \
  do {                                                                             \
    cudaError_t e_ = (call);                                                       \
    if (e_ != cudaSuccess)                                                         \
      return fail(CLOVER_ERR_CUDA, std::string(#call) + ": " + cudaGetErrorString(e_)); \
  } while (0)

#ifdef CLOVER_WITH_NCCL
#define NK(call)                                                                   \
  do {                                                                             \
    ncclResult_t r_ = (call);                                                      \
    if (r_ != ncclSuccess)                                                         \
      return fail(CLOVER_ERR_NCCL, std::string(#call) + ": " + ncclGetErrorString(r_)); \
  } while (0)
#endif

// Buffers of one chunk.  State A (time level 0), B (after the Lagrangian
// phase), C (after the first advection sweep); reset_field is the
// rotation C -> A performed by the second sweep writing into A.
// Buffers are carved in enum order at one common stride, so A + q (the five
// inputs of the Lagrangian phase, in the order of its staged rows LF_*) are
// one 3D tensor {pitch, rows, 5} for the TMA.
// The fused x sweeps read d1 e1 u1 v1 fy fx (sweep 1) and fx d2 e2 u2 v2
// (sweep 2) as one tensor each, so B is followed by fy, fx, then C.
enum Buf {
  B_D0, B_E0, B_U0, B_V0,     // A
  B_Q,
  B_D1, B_E1, B_U1, B_V1,     // B
  B_FY, B_FX,
  B_D2, B_E2, B_U2, B_V2,     // C
  B_MX, B_MY, B_SCR, NBUF
};
static_assert(B_E1 == B_D1 + XF<1>::E && B_U1 == B_D1 + XF<1>::U && B_V1 == B_D1 + XF<1>::V &&
                  B_FY == B_D1 + XF<1>::FY && B_FX == B_D1 + XF<1>::FX,
              "fused x sweep 1 tensor order");
static_assert(YRW == XRW && (int)YL<1>::E == XF<1>::E * YRW && (int)YL<1>::U == XF<1>::U * YRW &&
                  (int)YL<1>::V == XF<1>::V * YRW && (int)YL<1>::FY == XF<1>::FY * YRW &&
                  (int)YL<1>::FX == XF<1>::FX * YRW && B_E2 == B_D2 + 1 && B_U2 == B_D2 + 2 &&
                  B_V2 == B_D2 + 3,
              "fused y sweep tensors (sweep 1 shares the fused x sweep 1 map)");
static_assert(B_D2 == B_FX + XF<2>::R && B_E2 == B_FX + XF<2>::E && B_U2 == B_FX + XF<2>::U &&
                  B_V2 == B_FX + XF<2>::V,
              "fused x sweep 2 tensor order");
static_assert(B_E0 == B_D0 + VF_E && B_U0 == B_D0 + VF_U && B_V0 == B_D0 + VF_V,
              "visc tensor order");
static_assert(B_E0 == B_D0 + LF_E && B_U0 == B_D0 + LF_U && B_V0 == B_D0 + LF_V &&
                  B_Q == B_D0 + LF_Q, "Lagrangian tensor order");

const int kBufKind[NBUF] = {K_CELL, K_CELL, K_XVEL, K_YVEL, K_CELL,
                            K_CELL, K_CELL, K_XVEL, K_YVEL, K_YFACE, K_XFACE,
                            K_CELL, K_CELL, K_XVEL, K_YVEL,
                            K_XFACE, K_YFACE, K_CELL};

constexpr int64_t kAlign = 256;
inline int64_t align_up(int64_t v, int64_t a) { return (v + a - 1) / a * a; }

struct ChunkState {
  Chunk c;
  int cx, cy, id;
  double* buf[NBUF];
  double* partials;  // summary partials, ntx*nty*5
  int ntx, nty;
  FixSlot fix;       // warps to redo with IEEE division (clover_stream.cuh)
  FixSlot fix_b;     // the same for boundary segments running beside the interior (run_phase)
  CUtensorMap tm_lag;   // d0 e0 u0 v0 q as one {pitch, rows, 5} fp64 tensor, box {LRW, 1, 5}
  CUtensorMap tm_visc;  // d0 e0 u0 v0 as {pitch, rows, 4}, box {VRW, 1, 4}
  CUtensorMap tm_x1;    // d1 e1 u1 v1 fy fx, box {XRW, 1, 6} (fused y sweep 1)
  CUtensorMap tm_x1x;   // the same tensor, box {XRW, XBOX, 6} (fused x sweep 1)
  CUtensorMap tm_x2;    // fx d2 e2 u2 v2, box {XRW, 1, 5} (fused x sweep 2)
  CUtensorMap tm_fy;    // fy, box {YRW, 1, 1} (fused y sweep 2)
  CUtensorMap tm_c4;    // d2 e2 u2 v2, box {YRW, 1, 4} (fused y sweep 2)
  CUtensorMap tm_y2;    // fy fx d2 e2 u2 v2, box {YRW, 1, 6} (fused y sweep 2, CLOVER_Y2ONE)
};

struct Layout {
  int px, py;
  std::vector<int> xs, ys;  // chunk boundaries in global cells (size px+1, py+1)
  bool tile_aligned;
};

Layout decompose(int NX, int NY, int px, int py) {
  Layout L;
  L.px = px; L.py = py;
  L.tile_aligned = (NX >= ST * px) && (NY >= ST * py);
  auto split = [&](int N, int p, std::vector<int>& b) {
    b.assign(p + 1, 0);
    for (int i = 1; i < p; ++i) {
      int64_t v = (int64_t)i * N / p;
      if (L.tile_aligned) v = (v + ST / 2) / ST * ST;
      b[i] = (int)v;
    }
    b[p] = N;
  };
  split(NX, px, L.xs);
  split(NY, py, L.ys);
  return L;
}

int64_t field_elems(int nx, int ny, int* pitch_out) {
  // columns: j in [-COL0, nx+1+HALO_COLS] (at least) with j=0 at COL0;
  // rows k in [-HALO_ROWS, ny+1+HALO_ROWS]
  int pitch = (int)align_up(COL0 + nx + 2 + HALO_COLS, 32);
  if (pitch_out) *pitch_out = pitch;
  int rows = ny + 2 + 2 * HALO_ROWS;
  return (int64_t)pitch * rows;
}

// Fix-list capacity of a chunk: the most warps any step kernel's grid has
// (grid shapes as in enqueue_step).
inline int cdiv(int a, int b) { return (a + b - 1) / b; }
dim3 grid_cols(int ncols, int nrows, int ks) { return dim3(cdiv(ncols, SB), cdiv(nrows, ks)); }
// visc_dt's grid (blocks of SBV threads, one column per thread)
dim3 grid_cols_v(int ncols, int nrows, int ks) { return dim3(cdiv(ncols, SBV), cdiv(nrows, ks)); }
dim3 grid_strip(int ncols, int width, int nrows, int ks) {
  return dim3(cdiv(cdiv(ncols, width), SB / 32), cdiv(nrows, ks));
}
// Rows per segment: the compile-time default, halved (down to MIN_KS) while
// the grid would not fill the GPU once (148 SMs x SEG_FILL blocks): on small
// meshes shorter segments halve each block's row chain, the latency that
// bounds the step there.  Never below MIN_KS (fix-list capacity).
constexpr int MIN_KS = 8;
#ifndef CLOVER_SEG_FILL
#define CLOVER_SEG_FILL (8 * 64 / CLOVER_SB)  // blocks per SM: 16 warps/SM, as tuned on 2-warp blocks
#endif
int seg_rows(int ks, int64_t colblocks, int nrows) {
  while (ks > MIN_KS && colblocks * cdiv(nrows, ks) < 148 * CLOVER_SEG_FILL) ks /= 2;
  return ks;
}
// Segment rows of a kernel grid whose first nb segments have ks rows and
// the rest ks/2 (seg_rows_of).
// Full-height segments: all but about CLOVER_TAIL_WAVES waves of blocks
// (slots resident blocks on the GPU, colblocks blocks per segment row),
// which run at 1/CLOVER_TAIL_DIV height so the kernel's tail shrinks.
// Measured at 3840^2 (step ms, one box): none 0.965, 1 wave at 1/2 0.931,
// 2 waves at 1/2 0.925, 1 wave at 1/4 0.948, 2 waves at 1/4 0.938.
// CLOVER_TAIL=0: all full height.
#ifndef CLOVER_TAIL
#define CLOVER_TAIL 1
#endif
#ifndef CLOVER_TAIL_WAVES
#define CLOVER_TAIL_WAVES 2
#endif
int tail_nb(int ks, int64_t colblocks, int rows, int64_t slots, int td = CLOVER_TAIL_DIV) {
  if (!CLOVER_TAIL || ks < 4 * td || slots <= 0) return 0x3fffffff;
  const int64_t tail_rows = (int64_t)CLOVER_TAIL_WAVES *
                            cdiv((int)std::min<int64_t>(slots, 1 << 30), (int)colblocks) *
                            (int64_t)(ks / td);
  if (rows <= tail_rows) return 0;
  return (int)((rows - tail_rows) / ks);
}
// Deep halos (deep_ok below): state exchange depth, row extension of each
// phase's view beyond the chunk, minimum chunk height.
constexpr int DEEP_ROWS = 7;
constexpr int DEEP_EXT_VISC = 5, DEEP_EXT_LAGR = 5, DEEP_EXT_X1 = 4, DEEP_EXT_Y1 = 1;
constexpr int DEEP_EXT_MAX = 5;
constexpr int DEEP_MIN_NY = 16;
static_assert(DEEP_ROWS + 1 <= HALO_ROWS, "deep state halo allocated");
// (fix lists hold every warp segment of the largest kernel grid, views
// included: callers pass ny + 2 * DEEP_EXT_MAX)
int64_t fix_capacity(int nx, int ny) {
  // (adaptive segments: tail segments have at least 4 rows, see tail_nb;
  // the band layout adds at most one shorter segment per band: bounded by
  // counting segments of 2 rows)
  const dim3 g[7] = {grid_strip(nx, LW, ny, 2),
                     grid_strip(nx, CW_X, ny, CKS),    grid_cols(nx, ny, CKS_Y),
                     grid_strip(nx + 1, MW_X, ny + 1, MKS), grid_cols(nx + 1, ny + 1, MKS_Y),
                     grid_strip(nx + 1, XW, ny + 1, 2), grid_strip(nx + 1, YW, ny + 1, 2)};
  const dim3 gv = grid_cols_v(nx, ny, 2);  // visc_dt: SBV-thread blocks
  int64_t m = (int64_t)gv.x * gv.y * (SBV / 32);
  for (const dim3& d : g) m = std::max<int64_t>(m, (int64_t)d.x * d.y * (SB / 32));
  return m;
}
int64_t fix_bytes(int nx, int ny) { return kAlign + align_up(fix_capacity(nx, ny) * 8, kAlign); }

// cuTensorMapEncodeTiled through the runtime's driver entry point (no -lcuda).
typedef CUresult (*EncodeTiledFn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*,
                                  const cuuint64_t*, const cuuint64_t*, const cuuint32_t*,
                                  const cuuint32_t*, CUtensorMapInterleave, CUtensorMapSwizzle,
                                  CUtensorMapL2promotion, CUtensorMapFloatOOBfill);
EncodeTiledFn encode_tiled() {
  static EncodeTiledFn fn = nullptr;
  if (!fn) {
    void* p = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      fn = (EncodeTiledFn)p;
  }
  return fn;
}

// nf consecutive buffers of one chunk from `base` as a 3D fp64 tensor
// {pitch, rows, nf} (buffer stride fstride bytes); box {boxw, 1, nf} = one
// staged row of a kernel's ring.  Out-of-range columns (the last warp strip)
// read as zeros.
int encode_rows_map(CUtensorMap* m, const double* base, int pitch, int rows, int64_t fstride,
                    int nf, int boxw, int boxh = 1) {
  EncodeTiledFn fn = encode_tiled();
  if (!fn) return fail(CLOVER_ERR_CUDA, "cuTensorMapEncodeTiled unavailable");
  const cuuint64_t dims[3] = {(cuuint64_t)pitch, (cuuint64_t)rows, (cuuint64_t)nf};
  const cuuint64_t strides[2] = {(cuuint64_t)pitch * 8, (cuuint64_t)fstride};
  const cuuint32_t box[3] = {(cuuint32_t)boxw, (cuuint32_t)boxh, (cuuint32_t)nf};
  const cuuint32_t es[3] = {1, 1, 1};
  CUresult r = fn(m, CU_TENSOR_MAP_DATA_TYPE_FLOAT64, 3, (void*)base, dims, strides, box, es,
                  CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE,
                  CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) return fail(CLOVER_ERR_CUDA, "cuTensorMapEncodeTiled failed: " + std::to_string((int)r));
  return CLOVER_OK;
}

}  // namespace

struct clover_ctx {
  clover_grid g;
  std::vector<clover_state> states;
  int rank = 0, nranks = 1;
  Layout L;
  std::vector<ChunkState> chunks;  // local chunks
  std::vector<int> owner;          // chunk id -> rank
  cudaStream_t user = nullptr, work = nullptr;
  // halo exchanges run on `xs`: the work stream, or -- boundary segments
  // first, the interior overlapped with the exchange -- the comm stream
  cudaStream_t comm_stream = nullptr, xs = nullptr;
  cudaEvent_t ev_b = nullptr, ev_x = nullptr;
  bool overlap = false;  // see overlap_ok
  cudaEvent_t ev_in = nullptr, ev_out = nullptr;
  StepScalars* scal = nullptr;
  double* hist = nullptr;
  double* xbuf_send = nullptr;  // NCCL staging
  double* xbuf_recv = nullptr;
  int64_t xbuf_elems = 0;
  DtParams dtp;
  GlobalGeom gg;
  bool advect_x = true;
  bool use_graphs = true;
  bool fuse_x = true;  // fused x sweep where every chunk has both x walls (see fuse_x_ok)
  bool fuse_y = true;  // fused y sweep (see fuse_y_ok)
  bool fuse_y_chunks = true;  // ... also at y chunk boundaries (depth-4 row exchange)
  bool fuse_x_chunks = true;  // fused x sweep also at x chunk boundaries (depth-4 column exchange)
  // the y-wall band blocks may ride on a fixup launch (y_walls_after_fix)
  // only if every block of that launch is co-resident: the band blocks spin
  // until the fixup blocks are done (clover_init checks the occupancy)
  bool walls_fold_fits = false;
  bool deep = true;       // deep halos where they apply (deep_ok; clover_set_deep_halo)
  bool batch = true;      // several local chunks: one launch per kernel (KBatch; CLOVER_BATCH=0 off)
  bool chain = true;      // band layout of the row segments (seg_rows_lay; CLOVER_CHAIN=0 off)
  int nsm = 148, occ[4] = {1, 1, 1, 1};  // SMs, resident blocks/SM of the 4 segment kernels (set_segs)
  int state_rows = 0;     // rows of the state's y halo known current (ensure_state_rows)
  cudaGraphExec_t gexec[4] = {nullptr, nullptr, nullptr, nullptr};  // [parity + 2 * multi-step]
  int graph_launches[4] = {0, 0, 0, 0};  // kernels captured in gexec[i]
  int64_t launches = 0;  // step kernels launched so far (clover_launch_count)
  int64_t ws_bytes = 0;
  bool prof = false;
  bool virtual_remote = false;  // test mode: every chunk boundary takes the NCCL packing path
  bool virtual_nccl = false;    // ... and the messages travel through a 1-rank NCCL communicator
  std::vector<std::pair<int, cudaEvent_t>> prof_events;
#ifdef CLOVER_WITH_NCCL
  ncclComm_t comm = nullptr;
  // device-initiated halo stores (S:8(f) f1, lsa_setup): every rank's halo
  // mailbox is a symmetric NCCL window; a sender packs its boundary strips
  // straight into the receiver's mailbox through the peer mapping, then an
  // LSA barrier, the unpack, and a second barrier
  bool lsa = false;
  double* lsa_recv = nullptr;         // this rank's mailbox (ncclMemAlloc)
  size_t lsa_bytes = 0;
  ncclWindow_t lsa_win = nullptr;
  ncclDevComm lsa_dc{};
  bool lsa_dc_ok = false;
  std::vector<double*> lsa_peer;      // rank r's mailbox as mapped here
#endif
  int hist_first = 1;             // first step whose dt is in the history (after a restart: ckpt step + 1)
  bool use_ht = false;            // collectives through the caller's host transport
  clover_host_transport ht = {};
};

namespace {

void fill_defaults(clover_grid& g) {
  if (g.dtinit == 0.0) g.dtinit = 0.1;
  if (g.dtmax == 0.0) g.dtmax = 1.0;
  if (g.dtmin == 0.0) g.dtmin = 1.0e-7;
  if (g.dtrise == 0.0) g.dtrise = 1.5;
  if (g.dtc_safe == 0.0) g.dtc_safe = 0.7;
  if (g.dtu_safe == 0.0) g.dtu_safe = 0.5;
  if (g.dtv_safe == 0.0) g.dtv_safe = 0.5;
  if (g.dtdiv_safe == 0.0) g.dtdiv_safe = 0.7;
}

int validate(const clover_grid* g, const clover_dist* d, int* px, int* py, int* rank, int* nranks) {
  if (!g) return fail(CLOVER_ERR_ARG, "grid is NULL");
  if (g->x_cells < 4 || g->y_cells < 4) return fail(CLOVER_ERR_ARG, "x_cells and y_cells must be >= 4");
  if (!(g->xmax > g->xmin) || !(g->ymax > g->ymin)) return fail(CLOVER_ERR_ARG, "empty domain");
  if (g->face_mirror != 0 && g->face_mirror != 1) return fail(CLOVER_ERR_ARG, "face_mirror must be 0 or 1");
  *px = 1; *py = 1; *rank = 0; *nranks = 1;
  if (d) {
    *px = d->px; *py = d->py; *rank = d->rank; *nranks = d->nranks;
    if (*px < 1 || *py < 1) return fail(CLOVER_ERR_ARG, "px, py must be >= 1");
    if (*nranks < 1 || *rank < 0 || *rank >= *nranks) return fail(CLOVER_ERR_ARG, "bad rank/nranks");
    if ((*px * *py) % *nranks != 0) return fail(CLOVER_ERR_ARG, "px*py must be a multiple of nranks");
    if (*nranks > 1 && !d->nccl_unique_id && !d->host_transport)
      return fail(CLOVER_ERR_ARG, "nccl_unique_id or host_transport required for nranks > 1");
    if (d->host_transport && (!d->host_transport->sendrecv || !d->host_transport->allreduce_min_u64 ||
                              !d->host_transport->allgather_f64))
      return fail(CLOVER_ERR_ARG, "host_transport needs all three callbacks");
  }
  Layout L = decompose(g->x_cells, g->y_cells, *px, *py);
  for (int i = 0; i < *px; ++i)
    for (int jj = 0; jj < *py; ++jj)
      if (field_elems(L.xs[i + 1] - L.xs[i], L.ys[jj + 1] - L.ys[jj], nullptr) >= (int64_t)1 << 31)
        return fail(CLOVER_ERR_ARG, "a chunk field exceeds 2^31 elements: use more chunks");
  for (int i = 0; i < *px; ++i)
    if (L.xs[i + 1] - L.xs[i] < 4) return fail(CLOVER_ERR_ARG, "every chunk needs >= 4 cells in x");
  for (int i = 0; i < *py; ++i)
    if (L.ys[i + 1] - L.ys[i] < 4) return fail(CLOVER_ERR_ARG, "every chunk needs >= 4 cells in y");
  return CLOVER_OK;
}

std::vector<int> local_chunk_ids(int px, int py, int rank, int nranks) {
  int per = px * py / nranks;
  std::vector<int> ids;
  for (int i = rank * per; i < (rank + 1) * per; ++i) ids.push_back(i);
  return ids;
}

// Halo staging of one rank (doubles per buffer): every local chunk x 4
// sides x 6 fields x HALO_ROWS lines of the longest chunk extent.
int64_t staging_elems(const Layout& L, int rank, int nranks) {
  int64_t line = 0, n = 0;
  for (int id : local_chunk_ids(L.px, L.py, rank, nranks)) {
    const int cx = id % L.px, cy = id / L.px;
    const int nx = L.xs[cx + 1] - L.xs[cx], ny = L.ys[cy + 1] - L.ys[cy];
    line = std::max<int64_t>(line, std::max(ny + 2 + 2 * HALO_ROWS, nx + 2 + 2 * HALO_COLS));
    ++n;
  }
  return n * 4 * 6 * HALO_ROWS * line;
}

int64_t compute_workspace(const clover_grid* g, int px, int py, int rank, int nranks) {
  Layout L = decompose(g->x_cells, g->y_cells, px, py);
  int64_t bytes = align_up(sizeof(StepScalars), kAlign) + align_up(DT_HIST * 8, kAlign);
  int64_t maxrows = 0, maxcols = 0;
  for (int id : local_chunk_ids(px, py, rank, nranks)) {
    int cx = id % px, cy = id / px;
    int nx = L.xs[cx + 1] - L.xs[cx], ny = L.ys[cy + 1] - L.ys[cy];
    int64_t fe = field_elems(nx, ny, nullptr);
    bytes += NBUF * align_up(fe * 8, kAlign);
    int ntx = (nx + ST - 1) / ST, nty = (ny + ST - 1) / ST;
    bytes += align_up((int64_t)ntx * nty * 5 * 8, kAlign);
    bytes += 2 * fix_bytes(nx, ny + 2 * DEEP_EXT_MAX);
    maxrows = std::max<int64_t>(maxrows, ny + 2 + 2 * HALO_ROWS);
    maxcols = std::max<int64_t>(maxcols, nx + 2 + 2 * HALO_COLS);
  }
  if (px * py > 1) {
    // staging for the remote-neighbour path: every local chunk x 4 sides x
    // 6 fields x HALO_ROWS lines (also used by the virtual-remote test mode)
    int64_t line = std::max(maxrows, maxcols);
    int64_t el = (int64_t)local_chunk_ids(px, py, rank, nranks).size() * 4 * 6 * HALO_ROWS * line;
    bytes += 2 * align_up(el * 8, kAlign);
  }
  return bytes;
}

// ---------------------------------------------------------------- exchange
// Copy the halo strips of `fields` between neighbouring chunks: all x
// neighbours first (full allocated height, so y-halo rows travel too), then
// all y neighbours (full width, fixing the corners).  Local pairs use
// cudaMemcpy2DAsync; remote pairs NCCL send/recv through staging buffers.
struct XferDesc {  // one rectangular strip of one field
  double* base;    // chunk base (local (0,0))
  int pitch;
  int j0, k0, w, h;
};

inline double* strip_ptr(const XferDesc& d) { return d.base + (int64_t)d.k0 * d.pitch + d.j0; }

// Halo strips are many small rectangles (per phase: fields x sides x
// chunks, plus pack/unpack of the multi-GPU staging buffer); one
// cudaMemcpy2DAsync each cost ~2 us of launch per strip.  A batch collects
// the strips of one ordering stage and copies them in one kernel launch
// (elements enumerated strip by strip, rows contiguous for coalescing).
constexpr int MAX_STRIPS = 48;
struct StripCopy {
  double* dst;
  const double* src;
  int dpitch, spitch, w, h;
};
struct StripBatch {
  int n;
  long long start[MAX_STRIPS + 1];  // element offset of each strip; start[n] = total
  StripCopy s[MAX_STRIPS];
};
__global__ void __launch_bounds__(256) k_copy_strips(const __grid_constant__ StripBatch b) {
  const long long total = b.start[b.n];
  for (long long e = (long long)blockIdx.x * blockDim.x + threadIdx.x; e < total;
       e += (long long)gridDim.x * blockDim.x) {
    int lo = 0, hi = b.n - 1;  // last strip with start <= e
    while (lo < hi) {
      const int mid = (lo + hi + 1) >> 1;
      if (b.start[mid] <= e) lo = mid; else hi = mid - 1;
    }
    const StripCopy& c = b.s[lo];
    const long long off = e - b.start[lo];
    const int r = (int)(off / c.w), col = (int)(off - (long long)r * c.w);
    c.dst[(long long)r * c.dpitch + col] = c.src[(long long)r * c.spitch + col];
  }
}
struct StripQueue {
  clover_ctx* ctx;
  StripBatch b{};
  explicit StripQueue(clover_ctx* c) : ctx(c) { b.n = 0; b.start[0] = 0; }
  int add(double* dst, int dpitch, const double* src, int spitch, int w, int h);
  int add(const XferDesc& dst, const XferDesc& src) {
    return add(strip_ptr(dst), dst.pitch, strip_ptr(src), src.pitch, src.w, src.h);
  }
  int flush();
};

// strips for side `side` (0 left, 1 right, 2 bottom, 3 top) of chunk cs:
// send = owned points next to that side, recv = halo points of that side.
// x sides are `xdepth` columns deep, y sides `ydepth` rows: HALO, 4
// (HALO_COLS / FUSE_ROWS) for the inputs of a fused sweep across a chunk
// boundary, or DEEP_ROWS for the state with deep halos.
void side_strips(const ChunkState& cs, int buf, int side, XferDesc& send, XferDesc& recv,
                 int ydepth = HALO, int xdepth = HALO) {
  const Chunk& c = cs.c;
  const int kind = kBufKind[buf];
  const int ox = (kind == K_XVEL || kind == K_YVEL || kind == K_XFACE) ? 1 : 0;
  const int oy = (kind == K_XVEL || kind == K_YVEL || kind == K_YFACE) ? 1 : 0;
  send.base = recv.base = cs.buf[buf];
  send.pitch = recv.pitch = c.pitch;
  // full extent of this kind including both halos: rows [-HALO_ROWS,
  // ny+oy+HALO_ROWS], columns [-HALO_COLS, nx+ox+HALO_COLS] (x strips carry
  // every row, y strips every column, so 4-chunk corners are refreshed by
  // the second axis)
  const int full_h = c.ny + oy + 1 + 2 * HALO_ROWS, full_w = c.nx + ox + 1 + 2 * HALO_COLS;
  if (side == 0) {          // left: send [1+ox, d+ox], recv [1-d, 0]
    send.j0 = 1 + ox; recv.j0 = 1 - xdepth;
    send.w = recv.w = xdepth;
    send.k0 = recv.k0 = -HALO_ROWS; send.h = recv.h = full_h;
  } else if (side == 1) {   // right: send [nx+1-d, nx], recv [nx+ox+1, nx+ox+d]
    send.j0 = c.nx + 1 - xdepth; recv.j0 = c.nx + ox + 1;
    send.w = recv.w = xdepth;
    send.k0 = recv.k0 = -HALO_ROWS; send.h = recv.h = full_h;
  } else if (side == 2) {   // bottom: send [1+oy, d+oy], recv [1-d, 0]
    send.k0 = 1 + oy; recv.k0 = 1 - ydepth;
    send.h = recv.h = ydepth;
    send.j0 = recv.j0 = -HALO_COLS; send.w = recv.w = full_w;
  } else {                  // top: send [ny+1-d, ny], recv [ny+oy+1, ny+oy+d]
    send.k0 = c.ny + 1 - ydepth; recv.k0 = c.ny + oy + 1;
    send.h = recv.h = ydepth;
    send.j0 = recv.j0 = -HALO_COLS; send.w = recv.w = full_w;
  }
}

int neighbour(const clover_ctx* ctx, const ChunkState& cs, int side) {
  int cx = cs.cx, cy = cs.cy;
  if (side == 0) cx -= 1;
  if (side == 1) cx += 1;
  if (side == 2) cy -= 1;
  if (side == 3) cy += 1;
  if (cx < 0 || cy < 0 || cx >= ctx->L.px || cy >= ctx->L.py) return -1;
  return cy * ctx->L.px + cx;
}

ChunkState* local_chunk(clover_ctx* ctx, int id) {
  for (auto& cs : ctx->chunks)
    if (cs.id == id) return &cs;
  return nullptr;
}

int StripQueue::add(double* dst, int dpitch, const double* src, int spitch, int w, int h) {
  if (w <= 0 || h <= 0) return CLOVER_OK;
  if (b.n == MAX_STRIPS) {
    int rc = flush();
    if (rc) return rc;
  }
  b.s[b.n] = {dst, src, dpitch, spitch, w, h};
  b.start[b.n + 1] = b.start[b.n] + (long long)w * h;
  ++b.n;
  return CLOVER_OK;
}
int StripQueue::flush() {
  if (b.n == 0) return CLOVER_OK;
  const long long total = b.start[b.n];
  const int blocks = (int)std::min<long long>((total + 255) / 256, 148 * 8);
  k_copy_strips<<<blocks, 256, 0, ctx->xs>>>(b);
  CK(cudaGetLastError());
  b.n = 0;
  b.start[0] = 0;
  return CLOVER_OK;
}

// Geometry-only view of chunk `id` of the layout (any rank's): enough for
// neighbour() and the strip sizes of side_strips.
ChunkState geom_chunk(const clover_ctx* ctx, int id) {
  ChunkState g{};
  g.id = id; g.cx = id % ctx->L.px; g.cy = id / ctx->L.px;
  g.c.nx = ctx->L.xs[g.cx + 1] - ctx->L.xs[g.cx];
  g.c.ny = ctx->L.ys[g.cy + 1] - ctx->L.ys[g.cy];
  return g;
}
// Doubles of one side's message: the strips of every field in `bufs`.
int64_t msg_elems(const ChunkState& cs, int side, const std::vector<int>& bufs, int yd, int xd) {
  int64_t n = 0;
  for (int b : bufs) {
    XferDesc s, r;
    side_strips(cs, b, side, s, r, yd, xd);
    n += (int64_t)s.w * s.h;
  }
  return n;
}
// Where rank q receives the message of its chunk `id`, side `side`: the
// offset q's own message list (exchange_axis) gives it, rebuilt from the
// layout -- the address a sender stores into with device-initiated stores.
int64_t peer_recv_off(const clover_ctx* ctx, int q, int id, int side, const std::vector<int>& bufs,
                      int axis, int yd, int xd) {
  const int s_lo = axis == 0 ? 0 : 2, s_hi = axis == 0 ? 1 : 3;
  int64_t off = 0;
  for (int cid : local_chunk_ids(ctx->L.px, ctx->L.py, q, ctx->nranks)) {
    const ChunkState g = geom_chunk(ctx, cid);
    for (int sd : {s_lo, s_hi}) {
      const int nb = neighbour(ctx, g, sd);
      if (nb < 0 || (!ctx->virtual_remote && ctx->owner[nb] == q)) continue;
      if (cid == id && sd == side) return off;
      off += msg_elems(g, sd, bufs, yd, xd);
    }
  }
  return -1;
}

#ifdef CLOVER_WITH_NCCL
// LSA barrier over every rank of the node (one CTA; release/acquire at
// system scope): the device-initiated halo stores before it are visible to
// their receivers after it.
__global__ void k_lsa_barrier(ncclDevComm dc) {
  ncclLsaBarrierSession<ncclCoopCta> bar(ncclCoopCta(), dc, ncclTeamTagLsa(), 0);
  bar.sync(ncclCoopCta(), cuda::memory_order_acq_rel);
}
// rank r's window base as mapped into this process
__global__ void k_lsa_bases(ncclWindow_t w, int n, void** out) {
  for (int i = threadIdx.x; i < n; i += blockDim.x) out[i] = ncclGetPeerPointer(w, 0, i);
}
#endif
bool lsa_active(const clover_ctx* ctx) {
#ifdef CLOVER_WITH_NCCL
  return ctx->lsa && !ctx->use_ht && (ctx->nranks > 1 || (ctx->virtual_remote && ctx->virtual_nccl));
#else
  (void)ctx;
  return false;
#endif
}

// Device-initiated halo stores (S:8(f) f1): a symmetric NCCL window per rank
// as the halo mailbox (the same size on every rank: the largest rank's
// staging need), an LSA barrier, and the peers' mailbox addresses as mapped
// here.  Collective over the communicator: every rank calls it together.
int lsa_setup(clover_ctx* ctx) {
#ifdef CLOVER_WITH_NCCL
  if (ctx->lsa_recv) return CLOVER_OK;
  if (!ctx->comm) return fail(CLOVER_ERR_STATE, "LSA halo stores need an NCCL communicator");
  int64_t el = 0;
  for (int r = 0; r < ctx->nranks; ++r) el = std::max(el, staging_elems(ctx->L, r, ctx->nranks));
  ctx->lsa_bytes = (size_t)align_up(std::max<int64_t>(el * 8, 1), NCCL_WIN_REQUIRED_ALIGNMENT);
  NK(ncclMemAlloc((void**)&ctx->lsa_recv, ctx->lsa_bytes));
  NK(ncclCommWindowRegister(ctx->comm, ctx->lsa_recv, ctx->lsa_bytes, &ctx->lsa_win,
                            NCCL_WIN_COLL_SYMMETRIC));
  ncclDevCommRequirements reqs;
  std::memset(&reqs, 0, sizeof(reqs));
  reqs.lsaBarrierCount = 1;
  NK(ncclDevCommCreate(ctx->comm, &reqs, &ctx->lsa_dc));
  ctx->lsa_dc_ok = true;
  if (ncclTeamLsa(ctx->comm).nRanks != ctx->nranks)
    return fail(CLOVER_ERR_NCCL, "LSA halo stores need every rank load/store reachable (one NVLink domain)");
  void** d = nullptr;
  CK(cudaMalloc((void**)&d, sizeof(void*) * ctx->nranks));
  k_lsa_bases<<<1, 32, 0, ctx->work>>>(ctx->lsa_win, ctx->nranks, d);
  std::vector<void*> h((size_t)ctx->nranks);
  cudaError_t e = cudaMemcpyAsync(h.data(), d, sizeof(void*) * ctx->nranks, cudaMemcpyDeviceToHost,
                                  ctx->work);
  if (e == cudaSuccess) e = cudaStreamSynchronize(ctx->work);
  cudaFree(d);
  if (e != cudaSuccess) return fail(CLOVER_ERR_CUDA, std::string("LSA bases: ") + cudaGetErrorString(e));
  ctx->lsa_peer.assign((size_t)ctx->nranks, nullptr);
  for (int r = 0; r < ctx->nranks; ++r) ctx->lsa_peer[r] = (double*)h[r];
  return CLOVER_OK;
#else
  return fail(CLOVER_ERR_NCCL, "libclover built without NCCL");
#endif
}
void lsa_teardown(clover_ctx* ctx) {
#ifdef CLOVER_WITH_NCCL
  if (ctx->lsa_dc_ok) ncclDevCommDestroy(ctx->comm, &ctx->lsa_dc);
  if (ctx->lsa_win) ncclCommWindowDeregister(ctx->comm, ctx->lsa_win);
  if (ctx->lsa_recv) ncclMemFree(ctx->lsa_recv);
  ctx->lsa_dc_ok = false;
  ctx->lsa_win = nullptr;
  ctx->lsa_recv = nullptr;
  ctx->lsa = false;
#else
  (void)ctx;
#endif
}

int exchange_axis(clover_ctx* ctx, const std::vector<int>& bufs, int axis, int ydepth = HALO,
                  int xdepth = HALO) {
  const int s_lo = axis == 0 ? 0 : 2, s_hi = axis == 0 ? 1 : 3;
  // stage 1 (one batch): local pairs' halo strips and the packing of the
  // remote sides (owned points in, halo points / staging out: disjoint)
  StripQueue q(ctx);
  for (auto& cs : ctx->chunks) {
    if (ctx->virtual_remote) break;
    int nb = neighbour(ctx, cs, s_hi);
    if (nb < 0) continue;
    ChunkState* other = local_chunk(ctx, nb);
    if (!other) continue;
    for (int b : bufs) {
      XferDesc sA, rA, sB, rB;
      side_strips(cs, b, s_hi, sA, rA, ydepth, xdepth);
      side_strips(*other, b, s_lo, sB, rB, ydepth, xdepth);
      int rc = q.add(rB, sA);  // my high side -> neighbour's low halo
      if (rc) return rc;
      rc = q.add(rA, sB);      // neighbour's low side -> my high halo
      if (rc) return rc;
    }
  }
  if (ctx->nranks > 1 || ctx->virtual_remote) {
    // remote neighbours: pack every remote side into the staging buffer,
    // exchange all messages in one NCCL group, unpack.  In virtual-remote
    // mode (one process, test only) the NCCL pair is replaced by a device
    // copy from the partner message's send slot into this message's receive
    // slot; packing, offsets and unpacking are the NCCL path's own.
    struct Msg { int peer, nb; int64_t off, n; ChunkState* cs; int side; };
    std::vector<Msg> msgs;
    int64_t off = 0;
    for (auto& cs : ctx->chunks)
      for (int side : {s_lo, s_hi}) {
        int nb = neighbour(ctx, cs, side);
        if (nb < 0 || (!ctx->virtual_remote && local_chunk(ctx, nb))) continue;
        const int64_t n = msg_elems(cs, side, bufs, ydepth, xdepth);
        if (off + n > ctx->xbuf_elems) return fail(CLOVER_ERR_STATE, "halo staging buffer too small");
        msgs.push_back({ctx->owner[nb], nb, off, n, &cs, side});
        off += n;
      }
    // pack: into the staging buffer, or -- device-initiated stores (LSA) --
    // straight into the receiver's mailbox slot for this message
    const bool lsa = lsa_active(ctx);
    for (auto& m : msgs) {
      double* dst0 = ctx->xbuf_send + m.off;
#ifdef CLOVER_WITH_NCCL
      if (lsa) {
        const int64_t ro = peer_recv_off(ctx, m.peer, m.nb, m.side ^ 1, bufs, axis, ydepth, xdepth);
        if (ro < 0 || (size_t)(ro + m.n) * 8 > ctx->lsa_bytes)
          return fail(CLOVER_ERR_STATE, "LSA: no mailbox slot for a halo message");
        dst0 = ctx->lsa_peer[m.peer] + ro;
      }
#endif
      int64_t n = 0;
      for (int b : bufs) {
        XferDesc s, r;
        side_strips(*m.cs, b, m.side, s, r, ydepth, xdepth);
        XferDesc dst{dst0 + n, s.w, 0, 0, s.w, s.h};
        int rc = q.add(dst, s);
        if (rc) return rc;
        n += (int64_t)s.w * s.h;
      }
    }
    int rc = q.flush();  // the staging buffer is complete before it is sent
    if (rc) return rc;
    if (lsa) {
#ifdef CLOVER_WITH_NCCL
      // every sender's stores into this rank's mailbox are complete
      k_lsa_barrier<<<1, 128, 0, ctx->xs>>>(ctx->lsa_dc);
      if (cudaGetLastError() != cudaSuccess) return fail(CLOVER_ERR_CUDA, "LSA barrier launch failed");
#endif
    } else if (ctx->virtual_remote && ctx->virtual_nccl) {
#ifdef CLOVER_WITH_NCCL
      // one rank talks to itself: the i-th send to peer 0 matches the i-th
      // receive from peer 0, so each message's send is paired with the
      // receive slot of its partner (the neighbour's message on the facing
      // side), exactly as the two ranks' lists pair up in a real exchange
      NK(ncclGroupStart());
      for (auto& m : msgs) {
        const Msg* partner = nullptr;
        for (auto& pm : msgs)
          if (pm.cs->id == m.nb && pm.side == (m.side ^ 1)) partner = &pm;
        if (!partner || partner->n != m.n) return fail(CLOVER_ERR_STATE, "virtual remote: unmatched message");
        NK(ncclSend(ctx->xbuf_send + m.off, (size_t)m.n, ncclFloat64, 0, ctx->comm, ctx->xs));
        NK(ncclRecv(ctx->xbuf_recv + partner->off, (size_t)m.n, ncclFloat64, 0, ctx->comm, ctx->xs));
      }
      NK(ncclGroupEnd());
#else
      return fail(CLOVER_ERR_NCCL, "libclover built without NCCL");
#endif
    } else if (ctx->virtual_remote) {
      for (auto& m : msgs) {
        const Msg* partner = nullptr;
        for (auto& pm : msgs)
          if (pm.cs->id == m.nb && pm.side == (m.side ^ 1)) partner = &pm;
        if (!partner || partner->n != m.n) return fail(CLOVER_ERR_STATE, "virtual remote: unmatched message");
        rc = q.add(ctx->xbuf_recv + m.off, (int)m.n, ctx->xbuf_send + partner->off, (int)m.n, (int)m.n, 1);
        if (rc) return rc;
      }
      rc = q.flush();
      if (rc) return rc;
    } else if (ctx->use_ht) {
      // host transport: staging to host, the caller's sendrecv, back
      std::vector<double> hs((size_t)off), hr((size_t)off);
      CK(cudaMemcpyAsync(hs.data(), ctx->xbuf_send, (size_t)off * 8, cudaMemcpyDeviceToHost, ctx->xs));
      CK(cudaStreamSynchronize(ctx->xs));
      std::vector<int32_t> peer;
      std::vector<const double*> sp;
      std::vector<double*> rp;
      std::vector<int64_t> cnt;
      for (auto& m : msgs) {
        peer.push_back(m.peer);
        sp.push_back(hs.data() + m.off);
        rp.push_back(hr.data() + m.off);
        cnt.push_back(m.n);
      }
      if (ctx->ht.sendrecv(ctx->ht.user, (int32_t)msgs.size(), peer.data(), sp.data(), cnt.data(),
                           rp.data(), cnt.data()) != 0)
        return fail(CLOVER_ERR_NCCL, "host transport sendrecv failed");
      CK(cudaMemcpyAsync(ctx->xbuf_recv, hr.data(), (size_t)off * 8, cudaMemcpyHostToDevice, ctx->xs));
      CK(cudaStreamSynchronize(ctx->xs));
    } else {
#ifdef CLOVER_WITH_NCCL
      NK(ncclGroupStart());
      for (auto& m : msgs) {
        NK(ncclSend(ctx->xbuf_send + m.off, (size_t)m.n, ncclFloat64, m.peer, ctx->comm, ctx->xs));
        NK(ncclRecv(ctx->xbuf_recv + m.off, (size_t)m.n, ncclFloat64, m.peer, ctx->comm, ctx->xs));
      }
      NK(ncclGroupEnd());
#else
      return fail(CLOVER_ERR_NCCL, "libclover built without NCCL");
#endif
    }
    double* rbuf = ctx->xbuf_recv;
#ifdef CLOVER_WITH_NCCL
    if (lsa) rbuf = ctx->lsa_recv;
#endif
    for (auto& m : msgs) {
      int64_t n = 0;
      for (int b : bufs) {
        XferDesc s, r;
        side_strips(*m.cs, b, m.side, s, r, ydepth, xdepth);
        XferDesc src{rbuf + m.off + n, r.w, 0, 0, r.w, r.h};
        rc = q.add(r, src);
        if (rc) return rc;
        n += (int64_t)r.w * r.h;
      }
    }
#ifdef CLOVER_WITH_NCCL
    if (lsa) {
      // every rank has unpacked its mailbox before any sender stores the
      // next message into it
      rc = q.flush();
      if (rc) return rc;
      k_lsa_barrier<<<1, 128, 0, ctx->xs>>>(ctx->lsa_dc);
      if (cudaGetLastError() != cudaSuccess) return fail(CLOVER_ERR_CUDA, "LSA barrier launch failed");
      return CLOVER_OK;
    }
#endif
  }
  return q.flush();
}

bool needs_exchange(const clover_ctx* ctx) { return ctx->L.px * ctx->L.py > 1; }

int exchange(clover_ctx* ctx, const std::vector<int>& bufs, int ydepth = HALO, int xdepth = HALO) {
  if (!needs_exchange(ctx)) return CLOVER_OK;
  int rc = exchange_axis(ctx, bufs, 0, ydepth, xdepth);
  if (rc) return rc;
  return exchange_axis(ctx, bufs, 1, ydepth, xdepth);
}

// ---------------------------------------------------------------- schedule
dim3 cell_grid(const Chunk& c, int bx, int by) { return dim3((c.nx + bx - 1) / bx, (c.ny + by - 1) / by); }

#define LAUNCH_CHECK()                                                            \
  do {                                                                            \
    cudaError_t e_ = cudaGetLastError();                                          \
    if (e_ != cudaSuccess) return fail(CLOVER_ERR_CUDA, std::string("launch: ") + cudaGetErrorString(e_)); \
  } while (0)

#define STEP_LAUNCH_CHECK()                                                       \
  do {                                                                            \
    LAUNCH_CHECK();                                                               \
    ++ctx->launches;                                                              \
    if (ctx->prof) prof_mark(ctx, cur_prof_id);                                   \
  } while (0)
// after a fixup launch: its time joins the phase, it is not counted as a launch
constexpr int PROF_FIXUP = 0x100;
#define FIX_LAUNCH_CHECK()                                                        \
  do {                                                                            \
    LAUNCH_CHECK();                                                               \
    ++ctx->launches;                                                              \
    if (ctx->prof) prof_mark(ctx, cur_prof_id | PROF_FIXUP);                      \
  } while (0)

// Kernel types for clover_profile (names in kProfNames).
enum { P_VISC_DT, P_DT_FINAL, P_LAGR, P_CELL_X1, P_CELL_X2, P_CELL_Y1, P_CELL_Y2,
       P_MOM_X1, P_MOM_X2, P_MOM_Y1, P_MOM_Y2, P_ADV_X1, P_ADV_X2, P_ADV_Y1, P_ADV_Y2, NPROF };
const char* kProfNames[NPROF] = {"k_visc_dt", "k_dt_finalize", "k_lagrangian",
                                 "k_advec_cell_x<1>", "k_advec_cell_x<2>", "k_advec_cell_y<1>",
                                 "k_advec_cell_y<2>", "k_advec_mom_x<1>", "k_advec_mom_x<2>",
                                 "k_advec_mom_y<1>", "k_advec_mom_y<2>", "k_advec_x<1>",
                                 "k_advec_x<2>", "k_advec_y<1>", "k_advec_y<2>"};
static_assert(NPROF == CLOVER_PROFILE_SLOTS, "profile slots");

// Record an event after each profiled kernel; (prev event, this event)
// bracket exactly that kernel on the work stream.
void prof_mark(clover_ctx* ctx, int id) {
  cudaEvent_t e;
  cudaEventCreate(&e);
  cudaEventRecord(e, ctx->work);
  ctx->prof_events.push_back({id, e});
}


// Programmatic dependent launch (the kernels call pdl_trigger/pdl_wait,
// clover_common.cuh): launch latency and the next grid's block scheduling
// overlap the previous grid's tail; graph capture keeps the edges.  Used
// for the IEEE-fixup launches only (CLOVER_PDL_FIX): a streaming kernel
// launched early behind a fixup measured slower (same box, ms/step, PDL on
// streaming/fixup launches: on/on 0.8925, off/off 0.8905, off/on 0.8903 at
// 3840^2; 960^2 0.1495 / 0.1453 / 0.1435; 7680^2 3.26 / 3.24 / 3.24).
#ifndef CLOVER_PDL
#define CLOVER_PDL 0
#endif
#ifndef CLOVER_PDL_FIX
#define CLOVER_PDL_FIX 1
#endif
template <typename... KArgs, typename... Args>
cudaError_t launch_pdl(int pdl, void (*kernel)(KArgs...), dim3 grid, dim3 block, cudaStream_t st,
                       Args&&... args) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = grid;
  cfg.blockDim = block;
  cfg.dynamicSmemBytes = 0;
  cfg.stream = st;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  at[0].val.programmaticStreamSerializationAllowed = pdl;
  cfg.attrs = at;
  cfg.numAttrs = 1;
  return cudaLaunchKernelEx(&cfg, kernel, std::forward<Args>(args)...);
}
template <typename... KArgs, typename... Args>
cudaError_t launch_step(void (*kernel)(KArgs...), dim3 grid, dim3 block, cudaStream_t st,
                        Args&&... args) {
  return launch_pdl(CLOVER_PDL, kernel, grid, block, st, std::forward<Args>(args)...);
}
// IEEE-fixup launches (kf_*): their programmatic edge to the streaming
// kernel before them is set separately (CLOVER_PDL_FIX)
template <typename... KArgs, typename... Args>
cudaError_t launch_fix(void (*kernel)(KArgs...), dim3 grid, dim3 block, cudaStream_t st,
                       Args&&... args) {
  return launch_pdl(CLOVER_PDL_FIX, kernel, grid, block, st, std::forward<Args>(args)...);
}

// The fused x sweep (reach 4 columns along x) runs at x walls (mirrors of
// lanes of the same warp) and at x chunk boundaries (its inputs exchanged
// HALO_COLS deep, the neighbour's first columns recomputed); it needs the
// geometric face mirror.  fuse_x_chunks = false keeps the separate cell /
// momentum kernels at x chunk boundaries (A/B and tests).
bool fuse_x_ok(const clover_ctx* ctx) {
  if (!ctx->fuse_x || ctx->g.face_mirror == CLOVER_MIRROR_CELLCENTRE) return false;
  if (ctx->fuse_x_chunks) return true;
  for (const auto& cs : ctx->chunks)
    if (!cs.c.wl || !cs.c.wr) return false;
  return true;
}

// The fused y sweep (reach 4 rows along y) runs at y walls (the mirrored
// halo rows come from the band kernel) and at y chunk boundaries (its inputs
// exchanged FUSE_ROWS deep, the neighbour's first rows recomputed: SURVEY
// 8(e) H1/H2); it needs the geometric face mirror.  fuse_y_chunks = false
// keeps the separate cell / momentum kernels at y chunk boundaries (A/B and
// tests).
bool fuse_y_ok(const clover_ctx* ctx) {
  if (!ctx->fuse_y || ctx->g.face_mirror == CLOVER_MIRROR_CELLCENTRE) return false;
  if (ctx->fuse_y_chunks) return true;
  for (const auto& cs : ctx->chunks)
    if (!cs.c.wb || !cs.c.wt) return false;
  return true;
}

// ---------------------------------------------------------------- overlap
// Boundary segments first, the exchange overlapped with the interior
// (S:8(e) "boundary-strip-first + interior overlap"): for y-strip layouts
// (px == 1; x strips would need every row) whose exchanges leave the GPU
// (several ranks over NCCL) or take the remote path in virtual-remote mode.
// The host transport is synchronous, so it gains nothing there.
bool deep_ok(const clover_ctx* ctx);
bool overlap_ok(const clover_ctx* ctx) {
  return ctx->overlap && ctx->L.px == 1 && ctx->L.py > 1 && !ctx->use_ht &&
         (ctx->nranks > 1 || ctx->virtual_remote) && !deep_ok(ctx);
}

// ---------------------------------------------------------------- deep halos
// S:8(f) f1, communication-avoiding halos: the state (d0 e0 u0 v0) is
// exchanged once per step, DEEP_ROWS deep, and every kernel of the step runs
// over rows beyond its y chunk boundaries -- the rows of the neighbour it
// would otherwise receive -- so no other phase exchanges (the dt MIN stays).
// A kernel run on an extended view computes those rows with the same
// expressions from the same inputs as the neighbour does for its own rows:
// same bits, so the step stays bitwise equal to one chunk.  Extensions (rows
// beyond each non-wall y side), from the last reader back:
//   y sweep 2 (x-first step) reads its inputs rows -3 .. ny+4
//     -> x sweep 1 on rows -3 .. ny+4 (cells; nodes to ny+5): DEEP_EXT_X1 = 4
//   x sweep 2 (y-first step) reads rows 0 .. ny+1
//     -> y sweep 1 on rows 0 .. ny+1 (nodes to ny+2): DEEP_EXT_Y1 = 1
//   x sweep 1 on ext 4 reads rows -4 .. ny+6, y sweep 1 on ext 1 rows
//     -4 .. ny+5 -> the Lagrangian phase on ext 5 (cells -4 .. ny+5, nodes
//     and y faces to ny+6): DEEP_EXT_LAGR = 5
//   the Lagrangian on ext 5 reads q and the state rows -5 .. ny+7
//     -> visc_dt on ext 5 (q on its ring rows -5 and ny+6): DEEP_EXT_VISC = 5
//   visc_dt on ext 5 reads the state rows -6 .. ny+7: DEEP_ROWS = 7.
// The extra dt terms are the neighbours' own cells (the MIN is unchanged).
// y strips only (px == 1: every chunk has both x walls), both fused sweeps,
// chunks at least DEEP_MIN_NY rows (an extension never reaches past the
// neighbour).
bool deep_ok(const clover_ctx* ctx) {
  if (!ctx->deep || ctx->L.px != 1 || ctx->L.py < 2 || !fuse_x_ok(ctx) || !fuse_y_ok(ctx))
    return false;
  for (int k = 0; k < ctx->L.py; ++k)
    if (ctx->L.ys[k + 1] - ctx->L.ys[k] < DEEP_MIN_NY) return false;
  return true;
}

// Serpentine segment order: each step kernel reads what the previous one
// wrote, so alternate kernels run their row segments top-down (seg_y) and
// start on the rows still in L2: visc_dt and sweep 1 reversed, the
// Lagrangian phase and sweep 2 forward.  Measured at 3840^2: no gain
// (visc_dt +0.004 ms, Lagrangian -0.002 ms), so off by default.
#ifndef CLOVER_SERP
#define CLOVER_SERP 0
#endif
// Several local chunks: each streaming kernel and its fixup is one launch
// for all of them (KBatch, blockIdx.z = chunk; forward segment order).
bool batch_ok(const clover_ctx* ctx) {
  return ctx->batch && CLOVER_SERP == 0 && ctx->chunks.size() > 1 &&
         ctx->chunks.size() <= (size_t)MAX_BATCH;
}

// Row-segment parameters of a chunk (or view) of c.ny rows (see seg_rows,
// tail_nb): occ = resident blocks per SM of visc_dt, the Lagrangian, the
// fused x and y sweeps.
// Band layout (seg_rows_lay): one band per segment row of blocks resident
// at a time (ceil(slots / column blocks)), so a band's consecutive segments
// run in consecutive waves and share their overlap rows through L2; each
// band ends in CLOVER_TAIL_WAVES half-height segments (the kernel's last
// waves).  Used when every band holds at least one full segment and the
// tail; otherwise (small meshes, CLOVER_TAIL=0) the row layout (tail_nb).
// Env CLOVER_CHAIN=0 (read at init; default CLOVER_CHAIN): row layout.
// CLOVER_CHAIN_ADJ: bands added to that count (A/B builds).
#ifndef CLOVER_CHAIN
#define CLOVER_CHAIN 1
#endif
// Tail segments per kernel: ks / td rows (visc_dt, Lagrangian, x sweep,
// y sweep).  Quarter-height tails measured faster for visc_dt and the x
// sweeps, half-height for the Lagrangian and the y sweeps.
#ifndef CLOVER_TD_V
#define CLOVER_TD_V 4
#endif
#ifndef CLOVER_TD_L
#define CLOVER_TD_L 2
#endif
#ifndef CLOVER_TD_X
#define CLOVER_TD_X 4
#endif
#ifndef CLOVER_TD_Y
#define CLOVER_TD_Y 2
#endif
#ifndef CLOVER_CHAIN_ADJ
#define CLOVER_CHAIN_ADJ 0
#endif
void band_layout(bool on, int ks, int64_t colblocks, int rows, int64_t slots, int* ch, int* cf,
                 int td) {
  *ch = 0;
  *cf = 0;
  if (!on || !CLOVER_TAIL || ks < 4 * td || colblocks <= 0 || slots <= 0) return;
  const int64_t C = (slots + colblocks - 1) / colblocks + CLOVER_CHAIN_ADJ;
  if (C < 2 || C > rows) return;
  band_params(ks, (int)C, rows, ch, cf, td);
}

void set_segs(Chunk& c, int nsm, const int occ[4], bool chain) {
  c.vtd = CLOVER_TD_V; c.ltd = CLOVER_TD_L; c.xtd = CLOVER_TD_X; c.ytd = CLOVER_TD_Y;
  c.vks = seg_rows(VKS, grid_cols_v(c.nx, c.ny, VKS).x, c.ny);
  c.lks = seg_rows(LKS, grid_strip(c.nx, LW, c.ny, LKS).x, c.ny);
  c.xks = seg_rows(XKS, grid_strip(c.nx + 1, XW, c.ny + 1, XKS).x, c.ny + 1);
  c.yks = seg_rows(YKS, grid_strip(c.nx + 1, YW, c.ny + 1, YKS).x, c.ny + 1);
  // (short segments on small meshes: keep tail segments >= 4 rows)
  if (c.vks < 4 * c.vtd) c.vtd = CLOVER_TAIL_DIV;
  if (c.lks < 4 * c.ltd) c.ltd = CLOVER_TAIL_DIV;
  if (c.xks < 4 * c.xtd) c.xtd = CLOVER_TAIL_DIV;
  if (c.yks < 4 * c.ytd) c.ytd = CLOVER_TAIL_DIV;
  c.vnb = tail_nb(c.vks, grid_cols_v(c.nx, c.ny, c.vks).x, c.ny, (int64_t)nsm * occ[0], c.vtd);
  c.lnb = tail_nb(c.lks, grid_strip(c.nx, LW, c.ny, c.lks).x, c.ny, (int64_t)nsm * occ[1], c.ltd);
  c.xnb = tail_nb(c.xks, grid_strip(c.nx + 1, XW, c.ny + 1, c.xks).x, c.ny + 1, (int64_t)nsm * occ[2], c.xtd);
  c.ynb = tail_nb(c.yks, grid_strip(c.nx + 1, YW, c.ny + 1, c.yks).x, c.ny + 1, (int64_t)nsm * occ[3], c.ytd);
  band_layout(chain, c.vks, grid_cols_v(c.nx, c.ny, c.vks).x, c.ny, (int64_t)nsm * occ[0], &c.vch, &c.vcf,
              c.vtd);
  band_layout(chain, c.lks, grid_strip(c.nx, LW, c.ny, c.lks).x, c.ny, (int64_t)nsm * occ[1], &c.lch, &c.lcf,
              c.ltd);
  band_layout(chain, c.xks, grid_strip(c.nx + 1, XW, c.ny + 1, c.xks).x, c.ny + 1, (int64_t)nsm * occ[2],
              &c.xch, &c.xcf, c.xtd);
  band_layout(chain, c.yks, grid_strip(c.nx + 1, YW, c.ny + 1, c.yks).x, c.ny + 1, (int64_t)nsm * occ[3],
              &c.ych, &c.ycf, c.ytd);
}

// The chunk seen from `e` rows beyond each of its non-wall y sides: rows
// 1 .. ny+eb+et of the view are rows 1-eb .. ny+et of the chunk (field
// pointers and the TMA row origin shifted by eb rows).  Same fix lists.
ChunkState deep_view(const clover_ctx* ctx, const ChunkState& cs, int e) {
  ChunkState v = cs;
  Chunk& c = v.c;
  const int eb = c.wb ? 0 : e, et = c.wt ? 0 : e;
  c.ny += eb + et;
  c.gk0 -= eb;
  c.row0 = ROW0 - eb;
  for (int b = 0; b < NBUF; ++b) v.buf[b] = cs.buf[b] - (int64_t)eb * c.pitch;
  set_segs(c, ctx->nsm, ctx->occ, ctx->chain);
  return v;
}

// Row-segment geometry of a streaming kernel kind on a chunk: rows per
// segment, full-height segments, rows covered (seg_rows_of).
enum { SEG_LAGR, SEG_X, SEG_Y };
void seg_geom(const Chunk& c, int kind, int* ks, int* nb, int* rows, int* ch, int* cf, int* td) {
  if (kind == SEG_LAGR) { *ks = c.lks; *nb = c.lnb; *rows = c.ny; *ch = c.lch; *cf = c.lcf; *td = c.ltd; }
  else if (kind == SEG_X) { *ks = c.xks; *nb = c.xnb; *rows = c.ny + 1; *ch = c.xch; *cf = c.xcf; *td = c.xtd; }
  else { *ks = c.yks; *nb = c.ynb; *rows = c.ny + 1; *ch = c.ych; *cf = c.ycf; *td = c.ytd; }
}
// the segment holding row r (1-based), inverse of seg_rows_of
int seg_of_row(int r, int ks, int nb, int td) {
  if (r < 1) r = 1;
  if ((int64_t)(r - 1) < (int64_t)nb * ks) return (r - 1) / ks;
  return nb + (int)(((int64_t)(r - 1) - (int64_t)nb * ks) / (ks / td));
}
// Boundary / interior split of a chunk's segments [0, n) for an exchange of
// depth yd: [0, lo) holds the rows sent to the neighbour below (1 .. yd+1),
// [hi, n) those sent up (ny+1-yd .. ny); [lo, hi) is the interior.
void phase_ranges(const Chunk& c, int kind, int yd, int* lo, int* hi, int* n) {
  int ks, nb, rows, ch, cf, td;
  seg_geom(c, kind, &ks, &nb, &rows, &ch, &cf, &td);
  *n = seg_count_lay(ks, nb, ch, cf, rows, td);
  // (lo / hi: sub-range launches, row layout only -- callers pass ch = 0)
  *lo = c.wb ? 0 : std::min(*n, seg_of_row(yd + 1, ks, nb, td) + 1);
  *hi = c.wt ? *n : std::min(*n, std::max(*lo, seg_of_row(std::max(1, c.ny + 1 - yd), ks, nb, td)));
}

// Enqueue kernel phases [0, nphase) of one step (7 = full step).
// (Serpentine segment order, CLOVER_SERP: see batch_ok.)
static Chunk with_rev(Chunk c, int rev) {
  c.rev = rev;
  return c;
}

// The y-wall band work (YWalls) of advection sweep `sweep`, reading that
// sweep's inputs and writing its outputs.
static YWalls ywalls_of(const ChunkState& cs, int sweep) {
  YWalls y;
  y.nbx = cdiv(cs.c.nx + 2, SB);
  y.rho = cs.buf[sweep == 1 ? B_D1 : B_D2];
  y.en = cs.buf[sweep == 1 ? B_E1 : B_E2];
  y.fx = cs.buf[B_FX];
  y.fy = cs.buf[B_FY];
  y.rho_out = cs.buf[sweep == 1 ? B_D2 : B_D0];
  y.en_out = cs.buf[sweep == 1 ? B_E2 : B_E0];
  y.mfy = cs.buf[B_MY];
  return y;
}
static const YWalls kNoWalls = {0, nullptr, nullptr, nullptr, nullptr, nullptr, nullptr, nullptr};

int enqueue_step(clover_ctx* ctx, bool advect_x, int nphase) {
  cudaStream_t st = ctx->work;
  // one chunk on one rank: the y-wall bands ride on the fixup launch before
  // the y sweep (kf_lagrangian when sweep 1 is y, kf_advec_x<1> when sweep 2
  // is y), when that sweep is enqueued and fused
  const bool fold1 = ctx->chunks.size() == 1 && ctx->nranks == 1 && fuse_y_ok(ctx) &&
                     ctx->walls_fold_fits;
  const bool walls_in_lagr = CLOVER_YWALLS_FOLD && fold1 && !advect_x && nphase >= 4;
  const bool walls_in_x1 = CLOVER_YWALLS_FOLD && fold1 && advect_x && fuse_x_ok(ctx) && nphase >= 6;
  int cur_prof_id = P_VISC_DT;
  const bool deep = deep_ok(ctx);
  // several local chunks: one launch per kernel for all of them (KBatch)
  const bool batch = batch_ok(ctx);
  if (ctx->prof) prof_mark(ctx, -1);
  // one chunk on one rank: the visc fixup's last block finalises dt (no
  // k_dt_finalize launch); else the slot is combined first (NCCL MIN)
  const int fold_fin = (nphase >= 2 && ctx->chunks.size() == 1 && ctx->nranks == 1) ? 1 : 0;
  // A streaming kernel on every chunk, then the exchange of `bufs`.
  // launch(cs, c, n, stream, fix) runs the kernel over row segments
  // [c.seg0, c.seg0+n) on `stream`, pushing IEEE redos to `fix`;
  // fixup(cs, c, stream, fix) is its IEEE fixup.  With overlap_ok the
  // segments next to a y chunk boundary (the rows the exchange sends) run on
  // the comm stream, followed there by their fixup and the exchange, while
  // the interior segments run beside them on the work stream (own fix list);
  // the next phase waits for both.
  // ext > 0 (deep halos): the kernels run on each chunk's view extended
  // ext rows beyond its y chunk boundaries (deep_view); bufs may be empty.
  // batched (several local chunks, no overlap): launch_b(views) runs the
  // streaming kernel and its fixup once for all chunks (blockIdx.z = chunk).
  auto run_phase = [&](int kind, auto&& launch, auto&& fixup, auto&& launch_b,
                       const std::vector<int>& bufs, int yd, int xd, int ext = 0) -> int {
    if (batch && (ext > 0 || !overlap_ok(ctx))) {
      std::vector<ChunkState> views;
      views.reserve(ctx->chunks.size());
      for (auto& cs0 : ctx->chunks) views.push_back(ext > 0 ? deep_view(ctx, cs0, ext) : cs0);
      int rc = launch_b(views);
      if (rc) return rc;
      return bufs.empty() ? CLOVER_OK : exchange(ctx, bufs, yd, xd);
    }
    if (ext > 0 || !overlap_ok(ctx)) {
      for (auto& cs0 : ctx->chunks) {
        ChunkState view;
        ChunkState* csp = &cs0;
        if (ext > 0) {
          view = deep_view(ctx, cs0, ext);
          csp = &view;
        }
        ChunkState& cs = *csp;
        int lo, hi, n;
        phase_ranges(cs.c, kind, yd, &lo, &hi, &n);
        Chunk c = cs.c;
        c.seg0 = 0;
        int rc = launch(cs, c, n, st, cs.fix);
        if (!rc) rc = fixup(cs, c, st, cs.fix);
        if (rc) return rc;
      }
      return bufs.empty() ? CLOVER_OK : exchange(ctx, bufs, yd, xd);
    }
    cudaStream_t cm = ctx->comm_stream;
    CK(cudaEventRecord(ctx->ev_b, st));  // the previous phase is complete on st
    CK(cudaStreamWaitEvent(cm, ctx->ev_b, 0));
    std::vector<int> ilo(ctx->chunks.size()), ihi(ctx->chunks.size());
    for (size_t t = 0; t < ctx->chunks.size(); ++t) {
      auto& cs = ctx->chunks[t];
      int n;
      Chunk c = cs.c;
      c.vch = c.lch = c.xch = c.ych = 0;  // sub-range launches: row layout
      phase_ranges(c, kind, yd, &ilo[t], &ihi[t], &n);
      int rc = 0;
      bool any = false;
      if (ilo[t] > 0) { c.seg0 = 0; rc = launch(cs, c, ilo[t], cm, cs.fix_b); any = true; }
      if (!rc && ihi[t] < n) { c.seg0 = ihi[t]; rc = launch(cs, c, n - ihi[t], cm, cs.fix_b); any = true; }
      if (!rc && any) rc = fixup(cs, c, cm, cs.fix_b);
      if (rc) return rc;
    }
    ctx->xs = cm;
    int rc = exchange(ctx, bufs, yd, xd);
    ctx->xs = ctx->work;
    if (rc) return rc;
    CK(cudaEventRecord(ctx->ev_x, cm));
    for (size_t t = 0; t < ctx->chunks.size(); ++t) {
      if (ilo[t] >= ihi[t]) continue;
      auto& cs = ctx->chunks[t];
      Chunk c = cs.c;
      c.vch = c.lch = c.xch = c.ych = 0;
      c.seg0 = ilo[t];
      rc = launch(cs, c, ihi[t] - ilo[t], st, cs.fix);
      if (!rc) rc = fixup(cs, c, st, cs.fix);
      if (rc) return rc;
    }
    CK(cudaStreamWaitEvent(st, ctx->ev_x, 0));
    return CLOVER_OK;
  };
  if (nphase >= 1 && batch) {
    KBatch<VArgs> vb;
    dim3 g(1, 1, (unsigned)ctx->chunks.size());
    for (size_t t = 0; t < ctx->chunks.size(); ++t) {
      const ChunkState v = deep ? deep_view(ctx, ctx->chunks[t], DEEP_EXT_VISC) : ctx->chunks[t];
      vb.a[t].c = v.c;
      vb.a[t].tm = v.tm_visc;
      vb.a[t].q = v.buf[B_Q];
      vb.a[t].fix = v.fix;
      g.x = std::max(g.x, grid_cols_v(v.c.nx, v.c.ny, v.c.vks).x);
      g.y = std::max<unsigned>(g.y, (unsigned)seg_count_lay(v.c.vks, v.c.vnb, v.c.vch, v.c.vcf, v.c.ny, v.c.vtd));
    }
    launch_step(ks_visc_dt_b, g, SBV, st, vb, ctx->scal, ctx->dtp);
    STEP_LAUNCH_CHECK();
    launch_fix(kf_visc_dt_b, dim3(FIX_BLOCKS, 1, g.z), SBV, st, vb, ctx->scal, ctx->dtp);
    FIX_LAUNCH_CHECK();
    if (needs_exchange(ctx) && !deep) {
      int rc = exchange_axis(ctx, {B_Q}, 0);
      if (rc) return rc;
    }
    if (ctx->prof) prof_mark(ctx, -1);
  } else if (nphase >= 1) {
    for (auto& cs0 : ctx->chunks) {
      // deep halos: q (and the dt terms) of DEEP_EXT_VISC rows beyond the
      // chunk, the rows the Lagrangian view reads (no q exchange)
      ChunkState view;
      if (deep) view = deep_view(ctx, cs0, DEEP_EXT_VISC);
      const ChunkState& cs = deep ? view : cs0;
      const Chunk c = with_rev(cs.c, CLOVER_SERP);  // top-down: sweep 2 wrote these rows last
      launch_step(ks_visc_dt, dim3(grid_cols_v(c.nx, c.ny, c.vks).x, seg_count_lay(c.vks, c.vnb, c.vch, c.vcf, c.ny, c.vtd)), SBV, st, c, cs.tm_visc, cs.buf[B_Q],
                  ctx->scal, ctx->dtp, cs.fix);
      STEP_LAUNCH_CHECK();
      launch_fix(kf_visc_dt, FIX_BLOCKS, SBV, st, c, cs.tm_visc, cs.buf[B_Q], ctx->scal, ctx->dtp,
                  cs.fix, ctx->hist, fold_fin);
      FIX_LAUNCH_CHECK();
    }
    // q on ring 1: visc_dt computes rows 0 / ny+1 at y chunk boundaries
    // itself (visc_ring_rows); only x chunk boundaries exchange q
    if (needs_exchange(ctx) && !deep) {
      int rc = exchange_axis(ctx, {B_Q}, 0);
      if (rc) return rc;
    }
    if (ctx->prof) prof_mark(ctx, -1);
  }
  if (nphase >= 2) {
    cur_prof_id = P_DT_FINAL;
    if (ctx->nranks > 1 && ctx->use_ht) {
      uint64_t v = 0;
      CK(cudaMemcpyAsync(&v, &ctx->scal->dt_slot, 8, cudaMemcpyDeviceToHost, st));
      CK(cudaStreamSynchronize(st));
      if (ctx->ht.allreduce_min_u64(ctx->ht.user, &v) != 0)
        return fail(CLOVER_ERR_NCCL, "host transport allreduce failed");
      CK(cudaMemcpyAsync(&ctx->scal->dt_slot, &v, 8, cudaMemcpyHostToDevice, st));
      CK(cudaStreamSynchronize(st));
    }
#ifdef CLOVER_WITH_NCCL
    else if (ctx->nranks > 1 || ctx->virtual_nccl)
      NK(ncclAllReduce(&ctx->scal->dt_slot, &ctx->scal->dt_slot, 1, ncclUint64, ncclMin, ctx->comm, st));
#endif
    if (ctx->prof) prof_mark(ctx, -1);
    if (!fold_fin) {
      launch_step(k_dt_finalize, 1, 1, st, ctx->scal, ctx->hist, ctx->dtp);
      STEP_LAUNCH_CHECK();
    }
  }
  if (nphase >= 3) {
    cur_prof_id = P_LAGR;
    auto launch = [&](ChunkState& cs, Chunk c, int n, cudaStream_t sm, FixSlot fx) -> int {
      c = with_rev(c, 0);
      launch_step(ks_lagrangian, dim3(grid_strip(c.nx, LW, c.ny, c.lks).x, n), SB, sm, c, cs.tm_lag,
          cs.buf[B_D1], cs.buf[B_E1], cs.buf[B_U1], cs.buf[B_V1], cs.buf[B_FX], cs.buf[B_FY],
          ctx->scal, fx);
      STEP_LAUNCH_CHECK();
      return CLOVER_OK;
    };
    auto fixup = [&](ChunkState& cs, Chunk c, cudaStream_t sm, FixSlot fx) -> int {
      c = with_rev(c, 0);
      const YWalls yw = walls_in_lagr ? ywalls_of(cs, 1) : kNoWalls;
      launch_fix(kf_lagrangian, FIX_BLOCKS + 5 * yw.nbx, SB, sm, c, cs.tm_lag,
          cs.buf[B_D1], cs.buf[B_E1], cs.buf[B_U1], cs.buf[B_V1], cs.buf[B_FX], cs.buf[B_FY],
          ctx->scal, fx, yw);
      FIX_LAUNCH_CHECK();
      return CLOVER_OK;
    };
    auto launch_b = [&](std::vector<ChunkState>& vs) -> int {
      KBatch<LArgs> lb;
      dim3 g(1, 1, (unsigned)vs.size());
      for (size_t t = 0; t < vs.size(); ++t) {
        const ChunkState& v = vs[t];
        lb.a[t] = LArgs{v.c, v.tm_lag, v.buf[B_D1], v.buf[B_E1], v.buf[B_U1], v.buf[B_V1],
                        v.buf[B_FX], v.buf[B_FY], v.fix};
        g.x = std::max(g.x, grid_strip(v.c.nx, LW, v.c.ny, v.c.lks).x);
        g.y = std::max<unsigned>(g.y, (unsigned)seg_count_lay(v.c.lks, v.c.lnb, v.c.lch, v.c.lcf, v.c.ny, v.c.ltd));
      }
      launch_step(ks_lagrangian_b, g, SB, st, lb, ctx->scal);
      STEP_LAUNCH_CHECK();
      launch_fix(kf_lagrangian_b, dim3(FIX_BLOCKS, 1, g.z), SB, st, lb, ctx->scal);
      FIX_LAUNCH_CHECK();
      return CLOVER_OK;
    };
    // a fused y sweep (either sweep) reads these FUSE_ROWS deep in y; with
    // deep halos the phase runs DEEP_EXT_LAGR rows beyond the chunk instead
    int rc = deep ? run_phase(SEG_LAGR, launch, fixup, launch_b, {}, 0, 0, DEEP_EXT_LAGR)
                  : run_phase(SEG_LAGR, launch, fixup, launch_b,
                              {B_D1, B_E1, B_U1, B_V1, B_FX, B_FY},
                              fuse_y_ok(ctx) ? FUSE_ROWS : HALO, fuse_x_ok(ctx) ? HALO_COLS : HALO);
    if (rc) return rc;
    if (ctx->prof) prof_mark(ctx, -1);
  }
  // sweep 1 (direction d1) reads B writes C; sweep 2 reads C writes A.
  for (int sweep = 1; sweep <= 2; ++sweep) {
    const bool xdir = (sweep == 1) ? advect_x : !advect_x;
    const int ph_cell = sweep == 1 ? 4 : 6;
    const int rin = sweep == 1 ? B_D1 : B_D2, ein = sweep == 1 ? B_E1 : B_E2;
    const int rout = sweep == 1 ? B_D2 : B_D0, eout = sweep == 1 ? B_E2 : B_E0;
    const int uin = sweep == 1 ? B_U1 : B_U2, vin = sweep == 1 ? B_V1 : B_V2;
    const int uout = sweep == 1 ? B_U2 : B_U0, vout = sweep == 1 ? B_V2 : B_V0;
    const int mbuf = xdir ? B_MX : B_MY;
    if (xdir && fuse_x_ok(ctx)) {
      // advec_cell x + advec_mom x in one kernel (ks_advec_x): phase ph_cell
      // runs both, phase ph_cell + 1 is empty
      if (nphase >= ph_cell) {
        cur_prof_id = sweep == 1 ? P_ADV_X1 : P_ADV_X2;
        const int serp = sweep == 1 ? CLOVER_SERP : 0;
        auto launch = [&](ChunkState& cs, Chunk c, int n, cudaStream_t sm, FixSlot fx) -> int {
          c = with_rev(c, serp);
          const dim3 g(grid_strip(c.nx + 1, XW, c.ny + 1, c.xks).x, n);
          if (sweep == 1)
            launch_step(ks_advec_x<1>, g, SB, sm, c, cs.tm_x1x, cs.buf[rout], cs.buf[eout],
                        cs.buf[uout], cs.buf[vout], fx);
          else
            launch_step(ks_advec_x<2>, g, SB, sm, c, cs.tm_x2, cs.buf[rout], cs.buf[eout],
                        cs.buf[uout], cs.buf[vout], fx);
          STEP_LAUNCH_CHECK();
          return CLOVER_OK;
        };
        auto fixup = [&](ChunkState& cs, Chunk c, cudaStream_t sm, FixSlot fx) -> int {
          c = with_rev(c, serp);
          if (sweep == 1) {
            const YWalls yw = walls_in_x1 ? ywalls_of(cs, 2) : kNoWalls;
            launch_fix(kf_advec_x<1>, FIX_BLOCKS + 5 * yw.nbx, SB, sm, c, cs.tm_x1x, cs.buf[rout],
                        cs.buf[eout], cs.buf[uout], cs.buf[vout], fx, yw);
          } else {
            launch_fix(kf_advec_x<2>, FIX_BLOCKS, SB, sm, c, cs.tm_x2, cs.buf[rout], cs.buf[eout],
                        cs.buf[uout], cs.buf[vout], fx, kNoWalls);
          }
          FIX_LAUNCH_CHECK();
          return CLOVER_OK;
        };
        auto launch_b = [&](std::vector<ChunkState>& vs) -> int {
          KBatch<XArgs> xb;
          dim3 g(1, 1, (unsigned)vs.size());
          for (size_t t = 0; t < vs.size(); ++t) {
            const ChunkState& v = vs[t];
            xb.a[t] = XArgs{v.c, sweep == 1 ? v.tm_x1x : v.tm_x2, v.buf[rout], v.buf[eout],
                            v.buf[uout], v.buf[vout], v.fix};
            g.x = std::max(g.x, grid_strip(v.c.nx + 1, XW, v.c.ny + 1, v.c.xks).x);
            g.y = std::max<unsigned>(g.y, (unsigned)seg_count_lay(v.c.xks, v.c.xnb, v.c.xch, v.c.xcf, v.c.ny + 1, v.c.xtd));
          }
          if (sweep == 1) launch_step(ks_advec_x_b<1>, g, SB, st, xb);
          else launch_step(ks_advec_x_b<2>, g, SB, st, xb);
          STEP_LAUNCH_CHECK();
          if (sweep == 1) launch_fix(kf_advec_x_b<1>, dim3(FIX_BLOCKS, 1, g.z), SB, st, xb);
          else launch_fix(kf_advec_x_b<2>, dim3(FIX_BLOCKS, 1, g.z), SB, st, xb);
          FIX_LAUNCH_CHECK();
          return CLOVER_OK;
        };
        // sweep 1 feeds a fused y sweep 2: FUSE_ROWS deep in y.  Deep
        // halos: sweep 1 runs DEEP_EXT_X1 rows beyond the chunk (the rows the
        // y sweep 2 reads), sweep 2 ends the step with the one exchange
        int rc = !deep ? run_phase(SEG_X, launch, fixup, launch_b, {rout, eout, uout, vout},
                                   (sweep == 1 && fuse_y_ok(ctx)) ? FUSE_ROWS : HALO, HALO)
                 : sweep == 1 ? run_phase(SEG_X, launch, fixup, launch_b, {}, 0, 0, DEEP_EXT_X1)
                              : run_phase(SEG_X, launch, fixup, launch_b, {rout, eout, uout, vout},
                                          DEEP_ROWS, HALO);
        if (rc) return rc;
        if (ctx->prof) prof_mark(ctx, -1);
      }
      continue;
    }
    if (!xdir && fuse_y_ok(ctx)) {
      // advec_cell y on the wall bands of every chunk (rows 1..3, ny-1..ny,
      // mirrored), then advec_cell y + advec_mom y in one kernel
      // (ks_advec_y): phase ph_cell runs all, phase ph_cell + 1 is empty
      if (nphase >= ph_cell) {
        cur_prof_id = sweep == 1 ? P_ADV_Y1 : P_ADV_Y2;
        const bool folded = sweep == 1 ? walls_in_lagr : walls_in_x1;
        for (auto& cs : ctx->chunks) {
          if (folded) break;
          if (!cs.c.wb && !cs.c.wt) continue;  // no y wall band in this chunk
          const Chunk c = with_rev(cs.c, sweep == 1 ? CLOVER_SERP : 0);
          const YWalls yw = ywalls_of(cs, sweep);
          const dim3 gw(yw.nbx, 5);
          if (sweep == 1)
            launch_step(ks_cell_y_walls<1>, gw, SB, st, c, yw);
          else
            launch_step(ks_cell_y_walls<2>, gw, SB, st, c, yw);
          FIX_LAUNCH_CHECK();
        }
        const int serp = sweep == 1 ? CLOVER_SERP : 0;
        auto launch = [&](ChunkState& cs, Chunk c, int n, cudaStream_t sm, FixSlot fx) -> int {
          c = with_rev(c, serp);
          const dim3 g(grid_strip(c.nx + 1, YW, c.ny + 1, c.yks).x, n);
          const CUtensorMap& ta = sweep == 1 ? cs.tm_x1 : (CLOVER_Y2ONE ? cs.tm_y2 : cs.tm_fy);
          const CUtensorMap& tb = sweep == 1 ? cs.tm_x1 : (CLOVER_Y2ONE ? cs.tm_y2 : cs.tm_c4);
          if (sweep == 1) {
            launch_step(ks_advec_y<1>, g, SB, sm, c, ta, tb, cs.buf[rout], cs.buf[eout], cs.buf[B_MY],
                        cs.buf[uout], cs.buf[vout], fx);
          } else {
            launch_step(ks_advec_y<2>, g, SB, sm, c, ta, tb, cs.buf[rout], cs.buf[eout], cs.buf[B_MY],
                        cs.buf[uout], cs.buf[vout], fx);
          }
          STEP_LAUNCH_CHECK();
          return CLOVER_OK;
        };
        auto fixup = [&](ChunkState& cs, Chunk c, cudaStream_t sm, FixSlot fx) -> int {
          c = with_rev(c, serp);
          const CUtensorMap& ta = sweep == 1 ? cs.tm_x1 : (CLOVER_Y2ONE ? cs.tm_y2 : cs.tm_fy);
          const CUtensorMap& tb = sweep == 1 ? cs.tm_x1 : (CLOVER_Y2ONE ? cs.tm_y2 : cs.tm_c4);
          if (sweep == 1)
            launch_fix(kf_advec_y<1>, FIX_BLOCKS, SB, sm, c, ta, tb, cs.buf[rout], cs.buf[eout],
                        cs.buf[B_MY], cs.buf[uout], cs.buf[vout], fx);
          else
            launch_fix(kf_advec_y<2>, FIX_BLOCKS, SB, sm, c, ta, tb, cs.buf[rout], cs.buf[eout],
                        cs.buf[B_MY], cs.buf[uout], cs.buf[vout], fx);
          FIX_LAUNCH_CHECK();
          return CLOVER_OK;
        };
        // y sweep 1 feeds a fused x sweep 2: HALO_COLS deep in x.  Deep
        // halos: sweep 1 runs DEEP_EXT_Y1 rows beyond the chunk, sweep 2 ends
        // the step with the one exchange
        auto launch_b = [&](std::vector<ChunkState>& vs) -> int {
          KBatch<YArgs> yb;
          dim3 g(1, 1, (unsigned)vs.size());
          for (size_t t = 0; t < vs.size(); ++t) {
            const ChunkState& v = vs[t];
            yb.a[t] = YArgs{v.c, sweep == 1 ? v.tm_x1 : (CLOVER_Y2ONE ? v.tm_y2 : v.tm_fy),
                            sweep == 1 ? v.tm_x1 : (CLOVER_Y2ONE ? v.tm_y2 : v.tm_c4),
                            v.buf[rout], v.buf[eout], v.buf[B_MY], v.buf[uout], v.buf[vout],
                            v.fix};
            g.x = std::max(g.x, grid_strip(v.c.nx + 1, YW, v.c.ny + 1, v.c.yks).x);
            g.y = std::max<unsigned>(g.y, (unsigned)seg_count_lay(v.c.yks, v.c.ynb, v.c.ych, v.c.ycf, v.c.ny + 1, v.c.ytd));
          }
          if (sweep == 1) launch_step(ks_advec_y_b<1>, g, SB, st, yb);
          else launch_step(ks_advec_y_b<2>, g, SB, st, yb);
          STEP_LAUNCH_CHECK();
          if (sweep == 1) launch_fix(kf_advec_y_b<1>, dim3(FIX_BLOCKS, 1, g.z), SB, st, yb);
          else launch_fix(kf_advec_y_b<2>, dim3(FIX_BLOCKS, 1, g.z), SB, st, yb);
          FIX_LAUNCH_CHECK();
          return CLOVER_OK;
        };
        int rc = !deep ? run_phase(SEG_Y, launch, fixup, launch_b, {rout, eout, uout, vout}, HALO,
                                   (sweep == 1 && fuse_x_ok(ctx)) ? HALO_COLS : HALO)
                 : sweep == 1 ? run_phase(SEG_Y, launch, fixup, launch_b, {}, 0, 0, DEEP_EXT_Y1)
                              : run_phase(SEG_Y, launch, fixup, launch_b, {rout, eout, uout, vout},
                                          DEEP_ROWS, HALO);
        if (rc) return rc;
        if (ctx->prof) prof_mark(ctx, -1);
      }
      continue;
    }
    if (nphase >= ph_cell) {
      cur_prof_id = xdir ? (sweep == 1 ? P_CELL_X1 : P_CELL_X2) : (sweep == 1 ? P_CELL_Y1 : P_CELL_Y2);
      for (auto& cs : ctx->chunks) {
        const Chunk c = with_rev(cs.c, sweep == 1 ? CLOVER_SERP : 0);
        const double* fx = cs.buf[B_FX];
        const double* fy = cs.buf[B_FY];
        if (xdir) {
          const dim3 g = grid_strip(c.nx, CW_X, c.ny, CKS);
          if (sweep == 1) {
            launch_step(ks_advec_cell_x<1>, g, SB, st, c, cs.buf[rin], cs.buf[ein], fx, fy, cs.buf[rout], cs.buf[eout], cs.buf[mbuf], cs.fix);
            STEP_LAUNCH_CHECK();
            launch_fix(kf_advec_cell_x<1>, FIX_BLOCKS, SB, st, c, cs.buf[rin], cs.buf[ein], fx, fy, cs.buf[rout], cs.buf[eout], cs.buf[mbuf], cs.fix);
            FIX_LAUNCH_CHECK();
          } else {
            launch_step(ks_advec_cell_x<2>, g, SB, st, c, cs.buf[rin], cs.buf[ein], fx, fy, cs.buf[rout], cs.buf[eout], cs.buf[mbuf], cs.fix);
            STEP_LAUNCH_CHECK();
            launch_fix(kf_advec_cell_x<2>, FIX_BLOCKS, SB, st, c, cs.buf[rin], cs.buf[ein], fx, fy, cs.buf[rout], cs.buf[eout], cs.buf[mbuf], cs.fix);
            FIX_LAUNCH_CHECK();
          }
        } else {
          const dim3 g = grid_cols(c.nx, c.ny, CKS_Y);
          if (sweep == 1) {
            launch_step(ks_advec_cell_y<1>, g, SB, st, c, cs.buf[rin], cs.buf[ein], fx, fy, cs.buf[rout], cs.buf[eout], cs.buf[mbuf], cs.fix);
            STEP_LAUNCH_CHECK();
            launch_fix(kf_advec_cell_y<1>, FIX_BLOCKS, SB, st, c, cs.buf[rin], cs.buf[ein], fx, fy, cs.buf[rout], cs.buf[eout], cs.buf[mbuf], cs.fix);
            FIX_LAUNCH_CHECK();
          } else {
            launch_step(ks_advec_cell_y<2>, g, SB, st, c, cs.buf[rin], cs.buf[ein], fx, fy, cs.buf[rout], cs.buf[eout], cs.buf[mbuf], cs.fix);
            STEP_LAUNCH_CHECK();
            launch_fix(kf_advec_cell_y<2>, FIX_BLOCKS, SB, st, c, cs.buf[rin], cs.buf[ein], fx, fy, cs.buf[rout], cs.buf[eout], cs.buf[mbuf], cs.fix);
            FIX_LAUNCH_CHECK();
          }
        }
      }
      // x sweep 1 feeding a fused y sweep 2: the post-sweep density and
      // energy FUSE_ROWS deep in y; y sweep 1 feeding a fused x sweep 2:
      // HALO_COLS deep in x
      const int yd = (sweep == 1 && xdir && fuse_y_ok(ctx)) ? FUSE_ROWS : HALO;
      const int xd = (sweep == 1 && !xdir && fuse_x_ok(ctx)) ? HALO_COLS : HALO;
      int rc = exchange(ctx, {rout, eout, mbuf}, yd, xd);
      if (rc) return rc;
      if (ctx->prof) prof_mark(ctx, -1);
    }
    if (nphase >= ph_cell + 1) {
      cur_prof_id = xdir ? (sweep == 1 ? P_MOM_X1 : P_MOM_X2) : (sweep == 1 ? P_MOM_Y1 : P_MOM_Y2);
      for (auto& cs : ctx->chunks) {
        const Chunk c = with_rev(cs.c, sweep == 1 ? CLOVER_SERP : 0);
        if (xdir) {
          const dim3 g = grid_strip(c.nx + 1, MW_X, c.ny + 1, MKS);
          if (sweep == 1) {
            launch_step(ks_advec_mom_x<1>, g, SB, st, c, cs.buf[rout], cs.buf[mbuf], cs.buf[B_FY], cs.buf[uin], cs.buf[vin], cs.buf[uout], cs.buf[vout], cs.fix);
            STEP_LAUNCH_CHECK();
            launch_fix(kf_advec_mom_x<1>, FIX_BLOCKS, SB, st, c, cs.buf[rout], cs.buf[mbuf], cs.buf[B_FY], cs.buf[uin], cs.buf[vin], cs.buf[uout], cs.buf[vout], cs.fix);
            FIX_LAUNCH_CHECK();
          } else {
            launch_step(ks_advec_mom_x<2>, g, SB, st, c, cs.buf[rout], cs.buf[mbuf], cs.buf[B_FY], cs.buf[uin], cs.buf[vin], cs.buf[uout], cs.buf[vout], cs.fix);
            STEP_LAUNCH_CHECK();
            launch_fix(kf_advec_mom_x<2>, FIX_BLOCKS, SB, st, c, cs.buf[rout], cs.buf[mbuf], cs.buf[B_FY], cs.buf[uin], cs.buf[vin], cs.buf[uout], cs.buf[vout], cs.fix);
            FIX_LAUNCH_CHECK();
          }
        } else {
          const dim3 g = grid_cols(c.nx + 1, c.ny + 1, MKS_Y);
          if (sweep == 1) {
            launch_step(ks_advec_mom_y<1>, g, SB, st, c, cs.buf[rout], cs.buf[mbuf], cs.buf[B_FX], cs.buf[uin], cs.buf[vin], cs.buf[uout], cs.buf[vout], cs.fix);
            STEP_LAUNCH_CHECK();
            launch_fix(kf_advec_mom_y<1>, FIX_BLOCKS, SB, st, c, cs.buf[rout], cs.buf[mbuf], cs.buf[B_FX], cs.buf[uin], cs.buf[vin], cs.buf[uout], cs.buf[vout], cs.fix);
            FIX_LAUNCH_CHECK();
          } else {
            launch_step(ks_advec_mom_y<2>, g, SB, st, c, cs.buf[rout], cs.buf[mbuf], cs.buf[B_FX], cs.buf[uin], cs.buf[vin], cs.buf[uout], cs.buf[vout], cs.fix);
            STEP_LAUNCH_CHECK();
            launch_fix(kf_advec_mom_y<2>, FIX_BLOCKS, SB, st, c, cs.buf[rout], cs.buf[mbuf], cs.buf[B_FX], cs.buf[uin], cs.buf[vin], cs.buf[uout], cs.buf[vout], cs.fix);
            FIX_LAUNCH_CHECK();
          }
        }
      }
      const int yd = (sweep == 1 && xdir && fuse_y_ok(ctx)) ? FUSE_ROWS : HALO;
      const int xd = (sweep == 1 && !xdir && fuse_x_ok(ctx)) ? HALO_COLS : HALO;
      int rc = exchange(ctx, {uout, vout}, yd, xd);
      if (rc) return rc;
      if (ctx->prof) prof_mark(ctx, -1);
    }
  }
  return CLOVER_OK;
}

int join_in(clover_ctx* ctx) {
  CK(cudaEventRecord(ctx->ev_in, ctx->user));
  CK(cudaStreamWaitEvent(ctx->work, ctx->ev_in, 0));
  return CLOVER_OK;
}
int join_out(clover_ctx* ctx) {
  CK(cudaEventRecord(ctx->ev_out, ctx->work));
  CK(cudaStreamWaitEvent(ctx->user, ctx->ev_out, 0));
  return CLOVER_OK;
}

// Steps per multi-step graph: consecutive steps in one graph keep the
// programmatic (PDL) edges across the step boundary, which a graph launch
// per step breaks.
#ifndef CLOVER_GRAPH_STEPS
#define CLOVER_GRAPH_STEPS 1
#endif
// Graph of `nst` consecutive steps starting with sweep order `parity`
// (0: x first), instantiated into gexec[slot].
int build_graph(clover_ctx* ctx, int parity, int nst, int slot) {
  cudaGraph_t graph = nullptr;
  CK(cudaStreamBeginCapture(ctx->work, cudaStreamCaptureModeThreadLocal));
  int rc = 0;
  const int64_t n0 = ctx->launches;  // captured, not launched: counted per graph launch
  for (int i = 0; i < nst && !rc; ++i) rc = enqueue_step(ctx, (parity == 0) != (i % 2 == 1), 7);
  ctx->graph_launches[slot] = (int)(ctx->launches - n0);
  ctx->launches = n0;
  cudaError_t e = cudaStreamEndCapture(ctx->work, &graph);
  if (rc) {
    if (graph) cudaGraphDestroy(graph);
    return rc;
  }
  if (e != cudaSuccess) return fail(CLOVER_ERR_CUDA, std::string("capture: ") + cudaGetErrorString(e));
  e = cudaGraphInstantiate(&ctx->gexec[slot], graph, 0);
  cudaGraphDestroy(graph);
  if (e != cudaSuccess) return fail(CLOVER_ERR_CUDA, std::string("instantiate: ") + cudaGetErrorString(e));
  return CLOVER_OK;
}

// Wall mirrors and chunk halos of state fields written from outside a step
// (init, write_field, restart): DEEP_ROWS deep in y with deep halos.
int reflect_all(clover_ctx* ctx, const std::vector<int>& bufs) {
  for (auto& cs : ctx->chunks)
    for (int b : bufs) {
      dim3 blk(32, 8);
      dim3 grd((cs.c.nx + 2 + 2 * HALO + 31) / 32, (cs.c.ny + 2 + 2 * HALO + 7) / 8);
      k_reflect<<<grd, blk, 0, ctx->work>>>(cs.c, cs.buf[b], kBufKind[b]);
      LAUNCH_CHECK();
    }
  const int yd = deep_ok(ctx) ? DEEP_ROWS : HALO;
  int rc = exchange(ctx, bufs, yd, HALO);
  if (rc) return rc;
  if (bufs.size() == 4) ctx->state_rows = yd;
  else ctx->state_rows = std::min(ctx->state_rows, yd);
  return CLOVER_OK;
}

// A deep-halo step reads the state DEEP_ROWS deep; a step without deep halos
// (or a setting change since) left it HALO deep: refresh it first, outside
// any graph.
int ensure_state_rows(clover_ctx* ctx) {
  if (!deep_ok(ctx) || ctx->state_rows >= DEEP_ROWS) return CLOVER_OK;
  int rc = exchange(ctx, {B_D0, B_E0, B_U0, B_V0}, DEEP_ROWS, HALO);
  if (rc) return rc;
  ctx->state_rows = DEEP_ROWS;
  return CLOVER_OK;
}
// the state's halo depth after a full step
inline int step_state_rows(const clover_ctx* ctx) { return deep_ok(ctx) ? DEEP_ROWS : HALO; }

int check_err(clover_ctx* ctx) {
  CK(cudaStreamSynchronize(ctx->work));
  StepScalars h;
  CK(cudaMemcpy(&h, ctx->scal, sizeof(h), cudaMemcpyDeviceToHost));
  if (h.err == CLOVER_ERR_SMALL_DT) return fail(h.err, "small timestep: dt < dtmin");
  if (h.err == CLOVER_ERR_NEG_VOLUME) return fail(h.err, "negative volume (or NaN) in PdV");
  if (h.err) return fail(h.err, "latched device error");
  return CLOVER_OK;
}

struct FieldMap { int buf; int nxe_add, nye_add; };

int field_map(int fid, FieldMap* m) {
  switch (fid) {
    case CLOVER_F_DENSITY0: *m = {B_D0, 0, 0}; return 0;
    case CLOVER_F_ENERGY0: *m = {B_E0, 0, 0}; return 0;
    case CLOVER_F_PRESSURE: *m = {B_SCR, 0, 0}; return 0;
    case CLOVER_F_SOUNDSPEED: *m = {B_SCR, 0, 0}; return 0;
    case CLOVER_F_VISCOSITY: *m = {B_Q, 0, 0}; return 0;
    case CLOVER_F_XVEL0: *m = {B_U0, 1, 1}; return 0;
    case CLOVER_F_YVEL0: *m = {B_V0, 1, 1}; return 0;
    case CLOVER_F_VOL_FLUX_X: *m = {B_FX, 1, 0}; return 0;
    case CLOVER_F_VOL_FLUX_Y: *m = {B_FY, 0, 1}; return 0;
    case CLOVER_F_MASS_FLUX_X: *m = {B_MX, 1, 0}; return 0;
    case CLOVER_F_MASS_FLUX_Y: *m = {B_MY, 0, 1}; return 0;
  }
  return -1;
}

void kind_extra(int kind, int* ax, int* ay) {
  *ax = (kind == K_XVEL || kind == K_YVEL || kind == K_XFACE) ? 1 : 0;
  *ay = (kind == K_XVEL || kind == K_YVEL || kind == K_YFACE) ? 1 : 0;
}

// Gather buffer `buf` (global interior of its kind) into host.  Local chunks
// only; multi-rank gathers are done by the caller through NCCL.
int gather_local(clover_ctx* ctx, int buf, int kind, double* host, int64_t n) {
  int ax, ay;
  kind_extra(kind, &ax, &ay);
  const int NXE = ctx->g.x_cells + ax, NYE = ctx->g.y_cells + ay;
  if (n != (int64_t)NXE * NYE) return fail(CLOVER_ERR_ARG, "wrong element count for field");
  for (auto& cs : ctx->chunks) {
    const Chunk& c = cs.c;
    // owned range incl. the shared last node/face only on the global edge
    const int w = c.nx + ((c.gj0 + c.nx == ctx->g.x_cells) ? ax : 0);
    const int h = c.ny + ((c.gk0 + c.ny == ctx->g.y_cells) ? ay : 0);
    double* dst = host + (int64_t)c.gk0 * NXE + c.gj0;
    const double* src = cs.buf[buf] + idx(c, 1, 1);
    CK(cudaMemcpy2DAsync(dst, (size_t)NXE * 8, src, (size_t)c.pitch * 8, (size_t)w * 8, h,
                         cudaMemcpyDeviceToHost, ctx->work));
  }
  CK(cudaStreamSynchronize(ctx->work));
  return CLOVER_OK;
}

int scatter_local(clover_ctx* ctx, int buf, int kind, const double* host, int64_t n) {
  int ax, ay;
  kind_extra(kind, &ax, &ay);
  const int NXE = ctx->g.x_cells + ax, NYE = ctx->g.y_cells + ay;
  if (n != (int64_t)NXE * NYE) return fail(CLOVER_ERR_ARG, "wrong element count for field");
  for (auto& cs : ctx->chunks) {
    const Chunk& c = cs.c;
    const int w = c.nx + ax, h = c.ny + ay;  // owned incl. the shared last node
    const double* src = host + (int64_t)c.gk0 * NXE + c.gj0;
    double* dst = cs.buf[buf] + idx(c, 1, 1);
    CK(cudaMemcpy2DAsync(dst, (size_t)c.pitch * 8, src, (size_t)NXE * 8, (size_t)w * 8, h,
                         cudaMemcpyHostToDevice, ctx->work));
  }
  return CLOVER_OK;
}

// All-gather `count` doubles per rank (device `send`) into host `out`
// (nranks*count, rank-major).  Uses a temporary device buffer: this is the
// debug / I/O path (field readback, summaries, checkpoints), not the step.
int allgather_to_host(clover_ctx* ctx, const double* send, int64_t count, double* out) {
  if (ctx->use_ht) {
    std::vector<double> h((size_t)count);
    CK(cudaMemcpyAsync(h.data(), send, (size_t)count * 8, cudaMemcpyDeviceToHost, ctx->work));
    CK(cudaStreamSynchronize(ctx->work));
    if (ctx->ht.allgather_f64(ctx->ht.user, h.data(), count, out) != 0)
      return fail(CLOVER_ERR_NCCL, "host transport allgather failed");
    return CLOVER_OK;
  }
#ifdef CLOVER_WITH_NCCL
  double* recv = nullptr;
  CK(cudaMallocAsync((void**)&recv, (size_t)count * ctx->nranks * 8, ctx->work));
  ncclResult_t r = ncclAllGather(send, recv, (size_t)count, ncclFloat64, ctx->comm, ctx->work);
  cudaError_t e = cudaMemcpyAsync(out, recv, (size_t)count * ctx->nranks * 8, cudaMemcpyDeviceToHost, ctx->work);
  cudaFreeAsync(recv, ctx->work);
  if (r != ncclSuccess) return fail(CLOVER_ERR_NCCL, std::string("ncclAllGather: ") + ncclGetErrorString(r));
  if (e != cudaSuccess) return fail(CLOVER_ERR_CUDA, cudaGetErrorString(e));
  CK(cudaStreamSynchronize(ctx->work));
  return CLOVER_OK;
#else
  (void)ctx; (void)send; (void)count; (void)out;
  return fail(CLOVER_ERR_NCCL, "libclover built without NCCL");
#endif
}

// Owned block of chunk `id` for a field kind: global origin and extent (the
// shared last node/face column/row belongs to the chunk on the global edge).
void owned_block(const clover_ctx* ctx, int id, int ax, int ay, int* gj0, int* gk0, int* w, int* h) {
  const int cx = id % ctx->L.px, cy = id / ctx->L.px;
  *gj0 = ctx->L.xs[cx];
  *gk0 = ctx->L.ys[cy];
  const int nx = ctx->L.xs[cx + 1] - ctx->L.xs[cx], ny = ctx->L.ys[cy + 1] - ctx->L.ys[cy];
  *w = nx + ((ctx->L.xs[cx + 1] == ctx->g.x_cells) ? ax : 0);
  *h = ny + ((ctx->L.ys[cy + 1] == ctx->g.y_cells) ? ay : 0);
}

// Gather a field's global interior on every rank.  Single process: device to
// host copies.  Multi-rank: each rank packs its owned blocks (padded to the
// largest block) into one device buffer, NCCL all-gather, every rank unpacks
// all blocks into the host array.
int gather_all(clover_ctx* ctx, int buf, int kind, double* host, int64_t n) {
  if (ctx->nranks == 1) return gather_local(ctx, buf, kind, host, n);
  int ax, ay;
  kind_extra(kind, &ax, &ay);
  const int NXE = ctx->g.x_cells + ax, NYE = ctx->g.y_cells + ay;
  if (n != (int64_t)NXE * NYE) return fail(CLOVER_ERR_ARG, "wrong element count for field");
  int64_t maxblk = 0;
  for (int id = 0; id < ctx->L.px * ctx->L.py; ++id) {
    int gj, gk, w, h;
    owned_block(ctx, id, ax, ay, &gj, &gk, &w, &h);
    maxblk = std::max<int64_t>(maxblk, (int64_t)w * h);
  }
  const int64_t per = (int64_t)ctx->chunks.size() * maxblk;
  double* pack = nullptr;
  CK(cudaMallocAsync((void**)&pack, (size_t)per * 8, ctx->work));
  for (size_t t = 0; t < ctx->chunks.size(); ++t) {
    const ChunkState& cs = ctx->chunks[t];
    int gj, gk, w, h;
    owned_block(ctx, cs.id, ax, ay, &gj, &gk, &w, &h);
    CK(cudaMemcpy2DAsync(pack + t * maxblk, (size_t)w * 8, cs.buf[buf] + idx(cs.c, 1, 1),
                         (size_t)cs.c.pitch * 8, (size_t)w * 8, h, cudaMemcpyDeviceToDevice, ctx->work));
  }
  std::vector<double> all((size_t)per * ctx->nranks);
  int rc = allgather_to_host(ctx, pack, per, all.data());
  cudaFreeAsync(pack, ctx->work);
  if (rc) return rc;
  for (int r = 0; r < ctx->nranks; ++r) {
    const std::vector<int> ids = local_chunk_ids(ctx->L.px, ctx->L.py, r, ctx->nranks);
    for (size_t t = 0; t < ids.size(); ++t) {
      int gj, gk, w, h;
      owned_block(ctx, ids[t], ax, ay, &gj, &gk, &w, &h);
      const double* blk = all.data() + (size_t)r * per + t * maxblk;
      for (int k = 0; k < h; ++k)
        std::memcpy(host + (int64_t)(gk + k) * NXE + gj, blk + (int64_t)k * w, (size_t)w * 8);
    }
  }
  return CLOVER_OK;
}

// ---------------------------------------------------------------- checkpoint
// Access-execute analysis of one timestep (Fig. 8):
// each loop of the reference step with the datasets it reads
// (R) and writes (W); read-and-write counts as R.  Entering checkpoint mode
// before loop L, walk the (periodic) loop sequence from L: a dataset whose
// first access is a read must be saved, one whose first access is a write is
// dropped; datasets never written (mesh geometry) are not saved.
enum Dataset { D_RHO0, D_E0, D_U0, D_V0, D_P, D_CS, D_Q, D_RHO1, D_E1, D_U1, D_V1, D_FX, D_FY,
               D_MX, D_MY, ND };
#define DB(x) (1u << (x))
struct LoopAccess { const char* name; unsigned r, w; };
const LoopAccess kStepLoops[] = {
    {"ideal_gas", DB(D_RHO0) | DB(D_E0), DB(D_P) | DB(D_CS)},
    {"viscosity", DB(D_U0) | DB(D_V0) | DB(D_P) | DB(D_RHO0), DB(D_Q)},
    {"calc_dt", DB(D_CS) | DB(D_Q) | DB(D_RHO0) | DB(D_U0) | DB(D_V0), 0},
    {"PdV(predict)", DB(D_RHO0) | DB(D_E0) | DB(D_P) | DB(D_Q) | DB(D_U0) | DB(D_V0), DB(D_RHO1) | DB(D_E1)},
    {"ideal_gas(predict)", DB(D_RHO1) | DB(D_E1), DB(D_P) | DB(D_CS)},
    {"accelerate", DB(D_RHO0) | DB(D_P) | DB(D_Q) | DB(D_U0) | DB(D_V0), DB(D_U1) | DB(D_V1)},
    {"PdV(correct)", DB(D_RHO0) | DB(D_E0) | DB(D_P) | DB(D_Q) | DB(D_U0) | DB(D_V0) | DB(D_U1) | DB(D_V1),
     DB(D_RHO1) | DB(D_E1)},
    {"flux_calc", DB(D_U0) | DB(D_V0) | DB(D_U1) | DB(D_V1), DB(D_FX) | DB(D_FY)},
    {"advec_cell(1)", DB(D_RHO1) | DB(D_E1) | DB(D_FX) | DB(D_FY), DB(D_RHO1) | DB(D_E1) | DB(D_MX) | DB(D_MY)},
    {"advec_mom(1)", DB(D_RHO1) | DB(D_FX) | DB(D_FY) | DB(D_MX) | DB(D_MY) | DB(D_U1) | DB(D_V1),
     DB(D_U1) | DB(D_V1)},
    {"advec_cell(2)", DB(D_RHO1) | DB(D_E1) | DB(D_FX) | DB(D_FY), DB(D_RHO1) | DB(D_E1) | DB(D_MX) | DB(D_MY)},
    {"advec_mom(2)", DB(D_RHO1) | DB(D_FX) | DB(D_FY) | DB(D_MX) | DB(D_MY) | DB(D_U1) | DB(D_V1),
     DB(D_U1) | DB(D_V1)},
    {"reset_field", DB(D_RHO1) | DB(D_E1) | DB(D_U1) | DB(D_V1), DB(D_RHO0) | DB(D_E0) | DB(D_U0) | DB(D_V0)},
};
constexpr int kNumLoops = sizeof(kStepLoops) / sizeof(kStepLoops[0]);
#undef DB

unsigned checkpoint_plan(int loop) {
  unsigned decided = 0, save = 0;
  for (int t = 0; t < kNumLoops; ++t) {
    const LoopAccess& L = kStepLoops[(loop + t) % kNumLoops];
    const unsigned rnew = L.r & ~decided;
    save |= rnew;
    decided |= L.r | L.w;
  }
  return save;
}

constexpr uint64_t kCkptMagic = 0x54504b43564f4c43ull;  // "CLOVCKPT"
struct CkptHeader {
  uint64_t magic;
  int32_t version, x_cells, y_cells, face_mirror;
  int32_t step, advect_x, nfields, pad;
  double xmin, ymin, xmax, ymax, time, dt, dtold;
};

}  // namespace

// ====================================================================== C ABI
extern "C" {

int clover_abi_version(void) { return CLOVER_ABI_VERSION; }

const char* clover_last_error(void) { return g_last_error.c_str(); }

const char* clover_error_string(int code) {
  switch (code) {
    case CLOVER_OK: return "ok";
    case CLOVER_ERR_ARG: return "invalid argument";
    case CLOVER_ERR_CUDA: return "CUDA error";
    case CLOVER_ERR_NCCL: return "NCCL error";
    case CLOVER_ERR_WORKSPACE: return "workspace too small or misaligned";
    case CLOVER_ERR_SMALL_DT: return "small timestep (dt < dtmin)";
    case CLOVER_ERR_NEG_VOLUME: return "negative volume in PdV";
    case CLOVER_ERR_STATE: return "invalid state";
    case CLOVER_ERR_NAN: return "NaN in field_summary";
  }
  return "unknown error";
}

int clover_workspace_bytes(const clover_grid* grid, const clover_dist* dist, int64_t* bytes) {
  int px, py, rank, nranks;
  int rc = validate(grid, dist, &px, &py, &rank, &nranks);
  if (rc) return rc;
  if (!bytes) return fail(CLOVER_ERR_ARG, "bytes is NULL");
  *bytes = compute_workspace(grid, px, py, rank, nranks);
  return CLOVER_OK;
}

int clover_nccl_unique_id(void* out128) {
#ifdef CLOVER_WITH_NCCL
  if (!out128) return fail(CLOVER_ERR_ARG, "out is NULL");
  ncclUniqueId id;
  NK(ncclGetUniqueId(&id));
  static_assert(sizeof(ncclUniqueId) == 128, "ncclUniqueId size");
  std::memcpy(out128, &id, 128);
  return CLOVER_OK;
#else
  (void)out128;
  return fail(CLOVER_ERR_NCCL, "libclover built without NCCL");
#endif
}

int clover_init(const clover_grid* grid, const clover_state* states, int32_t nstates,
                const clover_dist* dist, void* workspace, int64_t workspace_bytes,
                void* cuda_stream, clover_ctx** out) {
  if (!out) return fail(CLOVER_ERR_ARG, "out is NULL");
  *out = nullptr;
  int px, py, rank, nranks;
  int rc = validate(grid, dist, &px, &py, &rank, &nranks);
  if (rc) return rc;
  if (!states || nstates < 1) return fail(CLOVER_ERR_ARG, "need at least one state");
  if (nstates > MAX_STATES) return fail(CLOVER_ERR_ARG, "too many states");
#ifndef CLOVER_WITH_NCCL
  if (nranks > 1 && !dist->host_transport) return fail(CLOVER_ERR_NCCL, "libclover built without NCCL");
#endif
  const int64_t need = compute_workspace(grid, px, py, rank, nranks);
  if (!workspace || workspace_bytes < need || ((uintptr_t)workspace % kAlign) != 0)
    return fail(CLOVER_ERR_WORKSPACE, "workspace must be >= clover_workspace_bytes and 256-B aligned");

  clover_ctx* ctx = new clover_ctx();
  ctx->g = *grid;
  fill_defaults(ctx->g);
  ctx->states.assign(states, states + nstates);
  ctx->rank = rank;
  ctx->nranks = nranks;
  ctx->L = decompose(grid->x_cells, grid->y_cells, px, py);
  ctx->user = (cudaStream_t)cuda_stream;
  ctx->ws_bytes = workspace_bytes;
  ctx->advect_x = ctx->g.advect_x_first != 0;
  ctx->dtp = DtParams{ctx->g.dtc_safe, ctx->g.dtu_safe, ctx->g.dtv_safe, ctx->g.dtdiv_safe,
                      ctx->g.dtrise, ctx->g.dtmax, ctx->g.dtmin};
  const double dx = (ctx->g.xmax - ctx->g.xmin) / (double)ctx->g.x_cells;
  const double dy = (ctx->g.ymax - ctx->g.ymin) / (double)ctx->g.y_cells;
  ctx->gg = GlobalGeom{ctx->g.x_cells, ctx->g.y_cells, ctx->g.xmin, ctx->g.ymin, dx, dy};

  auto bail = [&](int code) { clover_finalize(ctx); return code; };
  // boundary-first overlap: off by default (measured on one GPU, where all
  // chunks share the SMs, it only pays for 2-chunk layouts);
  // clover_debug_set_overlap or CLOVER_OVERLAP=1 turn it on
  ctx->overlap = false;
  if (const char* e = std::getenv("CLOVER_OVERLAP")) ctx->overlap = std::atoi(e) != 0;
  // deep halos where the layout allows (deep_ok; measured faster on every
  // y-strip layout): clover_set_deep_halo or CLOVER_DEEP_HALO=0
  ctx->deep = true;
  if (const char* e = std::getenv("CLOVER_DEEP_HALO")) ctx->deep = std::atoi(e) != 0;
  if (const char* e = std::getenv("CLOVER_BATCH")) ctx->batch = std::atoi(e) != 0;
  ctx->chain = CLOVER_CHAIN != 0;  // band layout (band_layout; CLOVER_CHAIN=0 off)
  if (const char* e = std::getenv("CLOVER_CHAIN")) ctx->chain = std::atoi(e) != 0;
  {
    int dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&ctx->nsm, cudaDevAttrMultiProcessorCount, dev);
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&ctx->occ[0], ks_visc_dt, SBV, 0);
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&ctx->occ[1], ks_lagrangian, SB, 0);
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&ctx->occ[2], ks_advec_x<1>, SB, 0);
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&ctx->occ[3], ks_advec_y<1>, SB, 0);
    cudaGetLastError();
  }
  if (cudaStreamCreateWithFlags(&ctx->work, cudaStreamNonBlocking) != cudaSuccess ||
      cudaStreamCreateWithFlags(&ctx->comm_stream, cudaStreamNonBlocking) != cudaSuccess ||
      cudaEventCreateWithFlags(&ctx->ev_b, cudaEventDisableTiming) != cudaSuccess ||
      cudaEventCreateWithFlags(&ctx->ev_x, cudaEventDisableTiming) != cudaSuccess ||
      cudaEventCreateWithFlags(&ctx->ev_in, cudaEventDisableTiming) != cudaSuccess ||
      cudaEventCreateWithFlags(&ctx->ev_out, cudaEventDisableTiming) != cudaSuccess)
    return bail(fail(CLOVER_ERR_CUDA, "stream/event creation failed"));

  ctx->xs = ctx->work;
  // carve the workspace
  char* p = (char*)workspace;
  ctx->scal = (StepScalars*)p;
  p += align_up(sizeof(StepScalars), kAlign);
  ctx->hist = (double*)p;
  p += align_up(DT_HIST * 8, kAlign);
  ctx->owner.assign(px * py, 0);
  for (int r = 0; r < nranks; ++r)
    for (int id : local_chunk_ids(px, py, r, nranks)) ctx->owner[id] = r;
  int64_t maxrows = 0, maxcols = 0;
  for (int id : local_chunk_ids(px, py, rank, nranks)) {
    ChunkState cs;
    cs.id = id; cs.cx = id % px; cs.cy = id / px;
    Chunk& c = cs.c;
    c.nx = ctx->L.xs[cs.cx + 1] - ctx->L.xs[cs.cx];
    c.ny = ctx->L.ys[cs.cy + 1] - ctx->L.ys[cs.cy];
    c.gj0 = ctx->L.xs[cs.cx];
    c.gk0 = ctx->L.ys[cs.cy];
    const int64_t fe = field_elems(c.nx, c.ny, &c.pitch);
    c.wl = cs.cx == 0; c.wr = cs.cx == px - 1; c.wb = cs.cy == 0; c.wt = cs.cy == py - 1;
    c.face_cc = ctx->g.face_mirror == CLOVER_MIRROR_CELLCENTRE;
    c.rev = 0;
    c.seg0 = 0;
    c.row0 = ROW0;
    set_segs(c, ctx->nsm, ctx->occ, ctx->chain);
    c.dx = dx; c.dy = dy; c.xmin = ctx->g.xmin; c.ymin = ctx->g.ymin;
    // correctly rounded reciprocals of the constant divisors (IEEE host division)
    c.rdx = 1.0 / dx; c.rdy = 1.0 / dy;
    c.r2dx = 1.0 / (dx + dx); c.r2dy = 1.0 / (dy + dy);
    c.rvol = 1.0 / (dx * dy); c.r2vol = 1.0 / (2.0 * (dx * dy));
    for (int b = 0; b < NBUF; ++b) {
      cs.buf[b] = (double*)p + (int64_t)ROW0 * c.pitch + COL0;
      p += align_up(fe * 8, kAlign);
    }
    {
      const double* base = cs.buf[B_D0] - (int64_t)ROW0 * c.pitch - COL0;
      const int rows = c.ny + 2 + 2 * HALO_ROWS;
      int rc = encode_rows_map(&cs.tm_lag, base, c.pitch, rows, align_up(fe * 8, kAlign), LNF, LRW, LBOX);
      const int64_t fs = align_up(fe * 8, kAlign);
      if (!rc) rc = encode_rows_map(&cs.tm_visc, base, c.pitch, rows, fs, VNF, VRW, VBOX);
      if (!rc) rc = encode_rows_map(&cs.tm_x1, base + (B_D1 - B_D0) * (fs / 8), c.pitch, rows, fs,
                                    XF<1>::NF, XRW);
      if (!rc) rc = encode_rows_map(&cs.tm_x1x, base + (B_D1 - B_D0) * (fs / 8), c.pitch, rows, fs,
                                    XF<1>::NF, XRW, XBOX);
      if (!rc) rc = encode_rows_map(&cs.tm_x2, base + (B_FX - B_D0) * (fs / 8), c.pitch, rows, fs,
                                    XF<2>::NF, XRW, XBOX);
      if (!rc) rc = encode_rows_map(&cs.tm_fy, base + (B_FY - B_D0) * (fs / 8), c.pitch, rows, fs,
                                    1, YRW);
      if (!rc) rc = encode_rows_map(&cs.tm_c4, base + (B_D2 - B_D0) * (fs / 8), c.pitch, rows, fs,
                                    4, YRW);
      if (!rc) rc = encode_rows_map(&cs.tm_y2, base + (B_FY - B_D0) * (fs / 8), c.pitch, rows, fs,
                                    6, YRW);
      if (rc) return bail(rc);
    }
    cs.ntx = (c.nx + ST - 1) / ST; cs.nty = (c.ny + ST - 1) / ST;
    cs.partials = (double*)p;
    p += align_up((int64_t)cs.ntx * cs.nty * 5 * 8, kAlign);
    cs.fix.hdr = (unsigned*)p;
    cs.fix.e = (uint2*)(p + kAlign);
    p += fix_bytes(c.nx, c.ny + 2 * DEEP_EXT_MAX);
    cs.fix_b.hdr = (unsigned*)p;
    cs.fix_b.e = (uint2*)(p + kAlign);
    p += fix_bytes(c.nx, c.ny + 2 * DEEP_EXT_MAX);
    maxrows = std::max<int64_t>(maxrows, c.ny + 2 + 2 * HALO_ROWS);
    maxcols = std::max<int64_t>(maxcols, c.nx + 2 + 2 * HALO_COLS);
    ctx->chunks.push_back(cs);
  }
  {
    // co-residency of the folded y-wall launches (kf_lagrangian, kf_advec_x<1>
    // with FIX_BLOCKS + 5 * nbx blocks): all blocks must fit at once
    int nsm = 148, dev = 0, b1 = 0, b2 = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b1, kf_lagrangian, SB, 0);
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b2, kf_advec_x<1>, SB, 0);
    cudaGetLastError();
    const int64_t resident = (int64_t)nsm * std::min(b1, b2);
    ctx->walls_fold_fits = ctx->chunks.size() == 1 &&
                           (int64_t)FIX_BLOCKS + 5 * ywalls_of(ctx->chunks[0], 1).nbx <= resident;
    if (const char* e = std::getenv("CLOVER_WALLS_FOLD_LIMIT"))  // test hook: force the unfolded path
      ctx->walls_fold_fits = ctx->walls_fold_fits && std::atoi(e) != 0;
  }
  if (px * py > 1) {
    int64_t line = std::max(maxrows, maxcols);
    ctx->xbuf_elems = (int64_t)ctx->chunks.size() * 4 * 6 * HALO_ROWS * line;
    ctx->xbuf_send = (double*)p;
    p += align_up(ctx->xbuf_elems * 8, kAlign);
    ctx->xbuf_recv = (double*)p;
    p += align_up(ctx->xbuf_elems * 8, kAlign);
  }
  if (nranks > 1 && dist->host_transport) {
    ctx->use_ht = true;
    ctx->ht = *dist->host_transport;
    ctx->use_graphs = false;  // host callbacks inside the step
  }
#ifdef CLOVER_WITH_NCCL
  if (nranks > 1 && !ctx->use_ht) {
    ncclUniqueId id;
    std::memcpy(&id, dist->nccl_unique_id, sizeof(id));
    if (ncclCommInitRank(&ctx->comm, nranks, id, rank) != ncclSuccess)
      return bail(fail(CLOVER_ERR_NCCL, "ncclCommInitRank failed"));
    // device-initiated halo stores over NVLink (CLOVER_LSA=1 on every rank)
    if (const char* e = std::getenv("CLOVER_LSA")) {
      if (std::atoi(e) != 0) {
        int rc = lsa_setup(ctx);
        if (rc) return bail(rc);
        ctx->lsa = true;
      }
    }
  }
#endif

  if (join_in(ctx)) return bail(CLOVER_ERR_CUDA);
  // zero every buffer (halo corners of unused kinds stay deterministic)
  if (cudaMemsetAsync(workspace, 0, (size_t)need, ctx->work) != cudaSuccess)
    return bail(fail(CLOVER_ERR_CUDA, "memset failed"));
  StepScalars h{};
  h.dt_slot = (unsigned long long)0;
  {
    double big = G_BIG;
    std::memcpy(&h.dt_slot, &big, 8);
  }
  h.dt = ctx->g.dtinit;
  h.dtold = ctx->g.dtinit;
  h.time = 0.0;
  h.step = 0;
  h.err = 0;
  if (cudaMemcpyAsync(ctx->scal, &h, sizeof(h), cudaMemcpyHostToDevice, ctx->work) != cudaSuccess)
    return bail(fail(CLOVER_ERR_CUDA, "scalar upload failed"));

  // states: rectangle edges nudged by dx/100 (reading A6), same expression as
  // the reference's read_input.
  StateList sl{};
  sl.n = nstates;
  for (int s = 0; s < nstates; ++s) {
    const clover_state& in = states[s];
    DevState& d = sl.s[s];
    d.density = in.density; d.energy = in.energy; d.xvel = in.xvel; d.yvel = in.yvel;
    d.geometry = in.geometry; d.xmin = in.xmin; d.xmax = in.xmax; d.ymin = in.ymin;
    d.ymax = in.ymax; d.radius = in.radius;
    if (s >= 1 && in.geometry == CLOVER_GEOM_RECT) {
      d.xmin = d.xmin + (dx / 100.0);
      d.ymin = d.ymin + (dy / 100.0);
      d.xmax = d.xmax - (dx / 100.0);
      d.ymax = d.ymax - (dy / 100.0);
    }
    if (s >= 1 && (in.geometry < 1 || in.geometry > 3))
      return bail(fail(CLOVER_ERR_ARG, "state geometry must be 1, 2 or 3"));
  }
  for (auto& cs : ctx->chunks) {
    dim3 blk(32, 8);
    dim3 grd((cs.c.nx + 2 + 2 * HALO + 31) / 32, (cs.c.ny + 2 + 2 * HALO + 7) / 8);
    k_generate<<<grd, blk, 0, ctx->work>>>(cs.c, ctx->gg, sl, cs.buf[B_D0], cs.buf[B_E0],
                                             cs.buf[B_U0], cs.buf[B_V0]);
    if (cudaGetLastError() != cudaSuccess) return bail(fail(CLOVER_ERR_CUDA, "k_generate launch"));
  }
  rc = reflect_all(ctx, {B_D0, B_E0, B_U0, B_V0});
  if (rc) return bail(rc);
  if (join_out(ctx)) return bail(CLOVER_ERR_CUDA);
  *out = ctx;
  return CLOVER_OK;
}

int clover_set_graphs(clover_ctx* ctx, int32_t enable) {
  if (!ctx) return fail(CLOVER_ERR_ARG, "ctx is NULL");
  ctx->use_graphs = enable != 0 && !ctx->use_ht;  // host callbacks cannot be captured
  return CLOVER_OK;
}

int clover_debug_set_virtual_remote(clover_ctx* ctx, int32_t enable) {
  if (!ctx) return fail(CLOVER_ERR_ARG, "ctx is NULL");
  if (ctx->nranks > 1) return fail(CLOVER_ERR_STATE, "virtual remote is a single-process test mode");
  if (enable && ctx->L.px * ctx->L.py < 2) return fail(CLOVER_ERR_STATE, "virtual remote needs px*py > 1");
  if (enable < 0 || enable > 3) return fail(CLOVER_ERR_ARG, "enable must be 0, 1, 2 or 3");
  if (enable >= 2) {
#ifdef CLOVER_WITH_NCCL
    if (!ctx->comm) {
      // a one-rank communicator on this GPU: every halo message becomes an
      // ncclSend/ncclRecv pair to self, the dt MIN a 1-rank ncclAllReduce
      CK(cudaStreamSynchronize(ctx->work));
      ncclUniqueId id;
      NK(ncclGetUniqueId(&id));
      NK(ncclCommInitRank(&ctx->comm, 1, id, 0));
    }
    if (enable == 3) {
      // device-initiated stores through a one-rank symmetric window: each
      // message is stored into its receiver's mailbox slot via the peer
      // mapping, LSA barriers around the unpack
      CK(cudaStreamSynchronize(ctx->work));
      int rc = lsa_setup(ctx);
      if (rc) return rc;
    }
    ctx->lsa = enable == 3;
#else
    return fail(CLOVER_ERR_NCCL, "libclover built without NCCL");
#endif
  }
  ctx->virtual_remote = enable != 0;
  ctx->virtual_nccl = enable >= 2;
  for (int i = 0; i < 4; ++i)
    if (ctx->gexec[i]) {
      cudaGraphExecDestroy(ctx->gexec[i]);
      ctx->gexec[i] = nullptr;
    }
  return CLOVER_OK;
}

int clover_set_deep_halo(clover_ctx* ctx, int32_t enable) {
  if (!ctx) return fail(CLOVER_ERR_ARG, "ctx is NULL");
  ctx->deep = enable != 0;
  for (int i = 0; i < 4; ++i)
    if (ctx->gexec[i]) {
      cudaGraphExecDestroy(ctx->gexec[i]);
      ctx->gexec[i] = nullptr;
    }
  return CLOVER_OK;  // the next step refreshes the state halo if needed (ensure_state_rows)
}

int clover_deep_halo_active(clover_ctx* ctx, int32_t* out) {
  if (!ctx || !out) return fail(CLOVER_ERR_ARG, "NULL argument");
  *out = deep_ok(ctx) ? 1 : 0;
  return CLOVER_OK;
}

int clover_debug_set_overlap(clover_ctx* ctx, int32_t enable) {
  if (!ctx) return fail(CLOVER_ERR_ARG, "ctx is NULL");
  ctx->overlap = enable != 0;
  for (int i = 0; i < 4; ++i)
    if (ctx->gexec[i]) {
      cudaGraphExecDestroy(ctx->gexec[i]);
      ctx->gexec[i] = nullptr;
    }
  return CLOVER_OK;
}

int clover_debug_set_fusion(clover_ctx* ctx, int32_t enable) {
  if (!ctx) return fail(CLOVER_ERR_ARG, "ctx is NULL");
  if (enable < 0 || enable > 2) return fail(CLOVER_ERR_ARG, "enable must be 0, 1 or 2");
  ctx->fuse_x = enable != 0;
  ctx->fuse_y = enable != 0;
  ctx->fuse_y_chunks = enable == 1;
  ctx->fuse_x_chunks = enable == 1;
  for (int i = 0; i < 4; ++i)
    if (ctx->gexec[i]) {
      cudaGraphExecDestroy(ctx->gexec[i]);
      ctx->gexec[i] = nullptr;
    }
  return CLOVER_OK;
}

int clover_debug_fix_count(clover_ctx* ctx, int64_t* out) {
  if (!ctx || !out) return fail(CLOVER_ERR_ARG, "NULL argument");
  CK(cudaStreamSynchronize(ctx->work));
  int64_t t = 0;
  for (auto& cs : ctx->chunks) {
    unsigned h[3];
    CK(cudaMemcpy(h, cs.fix.hdr, sizeof(h), cudaMemcpyDeviceToHost));
    t += h[2];
    CK(cudaMemcpy(h, cs.fix_b.hdr, sizeof(h), cudaMemcpyDeviceToHost));
    t += h[2];
  }
  *out = t;
  return CLOVER_OK;
}

int clover_kernels_per_step(clover_ctx* ctx, int32_t* out) {
  if (!ctx || !out) return fail(CLOVER_ERR_ARG, "NULL argument");
  // visc_dt + fixup, Lagrangian + fixup, the x sweep (fused: kernel + fixup;
  // else cell, mom + 2 fixups), the y sweep (fused: wall bands, kernel +
  // fixup; else 4; the bands ride on the previous fixup launch at one chunk
  // on one rank, enqueue_step) -- per chunk, or once for all local chunks
  // when batched (batch_ok; the unfused sweeps and the y-wall bands stay per
  // chunk) -- plus k_dt_finalize once unless the visc fixup finalises dt (one
  // chunk on one rank).  (Chunks without a y wall launch no band kernel; the
  // halo strip copies, k_copy_strips, are not counted.)
  const bool one = ctx->chunks.size() == 1 && ctx->nranks == 1;
  const bool folded = CLOVER_YWALLS_FOLD && one && fuse_x_ok(ctx) && ctx->walls_fold_fits;
  const bool bat = batch_ok(ctx), ov = overlap_ok(ctx);
  const int nch = (int)ctx->chunks.size();
  // boundary ranges + interior as separate launches, a fixup after each part
  // (run_phase with the boundary-first overlap)
  auto extra = [&](const ChunkState& cs, int kind, int yd) {
    int lo, hi, ns;
    Chunk c = cs.c;
    c.vch = c.lch = c.xch = c.ych = 0;  // overlap launches use the row layout
    phase_ranges(c, kind, yd, &lo, &hi, &ns);
    const int b = (lo > 0) + (hi < ns);
    return b + (b > 0) + 2 * (lo < hi) - 2;
  };
  // a fused phase: 2 launches, batched or per chunk (+ the overlap split)
  auto fused = [&](int kind, int yd) {
    if (bat && !ov) return 2;
    int m = 0;
    for (const auto& cs : ctx->chunks) m += 2 + (ov ? extra(cs, kind, yd) : 0);
    return m;
  };
  int n = one ? 0 : 1;
  n += bat ? 2 : 2 * nch;  // visc_dt
  n += fused(SEG_LAGR, fuse_y_ok(ctx) ? FUSE_ROWS : HALO);
  const bool ax = ctx->advect_x;
  for (int sweep = 1; sweep <= 2; ++sweep) {
    const bool xdir = (sweep == 1) ? ax : !ax;
    if (xdir) {
      n += fuse_x_ok(ctx) ? fused(SEG_X, (sweep == 1 && fuse_y_ok(ctx)) ? FUSE_ROWS : HALO) : 4 * nch;
    } else if (fuse_y_ok(ctx)) {
      for (const auto& cs : ctx->chunks) n += (!folded && (cs.c.wb || cs.c.wt)) ? 1 : 0;
      n += fused(SEG_Y, HALO);
    } else {
      n += 4 * nch;
    }
  }
  *out = (int32_t)n;
  return CLOVER_OK;
}

int clover_step(clover_ctx* ctx, int32_t nsteps) {
  if (!ctx) return fail(CLOVER_ERR_ARG, "ctx is NULL");
  if (nsteps < 0) return fail(CLOVER_ERR_ARG, "nsteps < 0");
  if (nsteps == 0) return CLOVER_OK;
  int rc = join_in(ctx);
  if (rc) return rc;
  // on an error after join_in, whatever was enqueued is still ordered before
  // later work on the caller's stream (join_out's own error is ignored)
  auto bail = [&](int code) {
    join_out(ctx);
    return code;
  };
  rc = ensure_state_rows(ctx);
  if (rc) return bail(rc);
  for (int i = 0; i < nsteps; ++i) {
    const int parity = ctx->advect_x ? 0 : 1;
    ctx->state_rows = step_state_rows(ctx);
    if (ctx->use_graphs && CLOVER_GRAPH_STEPS > 1 && nsteps - i >= CLOVER_GRAPH_STEPS) {
      const int slot = parity + 2;
      if (!ctx->gexec[slot]) {
        rc = build_graph(ctx, parity, CLOVER_GRAPH_STEPS, slot);
        if (rc) return bail(rc);
      }
      if (cudaGraphLaunch(ctx->gexec[slot], ctx->work) != cudaSuccess)
        return bail(fail(CLOVER_ERR_CUDA, "cudaGraphLaunch failed"));
      ctx->launches += ctx->graph_launches[slot];
      i += CLOVER_GRAPH_STEPS - 1;
      if (CLOVER_GRAPH_STEPS % 2) ctx->advect_x = !ctx->advect_x;
      continue;
    }
    if (ctx->use_graphs) {
      if (!ctx->gexec[parity]) {
        rc = build_graph(ctx, parity, 1, parity);
        if (rc) return bail(rc);
      }
      if (cudaGraphLaunch(ctx->gexec[parity], ctx->work) != cudaSuccess)
        return bail(fail(CLOVER_ERR_CUDA, "cudaGraphLaunch failed"));
      ctx->launches += ctx->graph_launches[parity];
    } else {
      rc = enqueue_step(ctx, ctx->advect_x, 7);
      if (rc) return bail(rc);
    }
    ctx->advect_x = !ctx->advect_x;
  }
  return join_out(ctx);
}

int clover_local_block(clover_ctx* ctx, int32_t* out4) {
  if (!ctx || !out4) return fail(CLOVER_ERR_ARG, "NULL argument");
  int j0 = 1 << 30, k0 = 1 << 30, j1 = 0, k1 = 0;
  for (const auto& cs : ctx->chunks) {
    j0 = std::min(j0, cs.c.gj0); k0 = std::min(k0, cs.c.gk0);
    j1 = std::max(j1, cs.c.gj0 + cs.c.nx); k1 = std::max(k1, cs.c.gk0 + cs.c.ny);
  }
  out4[0] = j0; out4[1] = k0; out4[2] = j1 - j0; out4[3] = k1 - k0;
  return CLOVER_OK;
}

int clover_launch_count(clover_ctx* ctx, int64_t* out) {
  if (!ctx || !out) return fail(CLOVER_ERR_ARG, "NULL argument");
  *out = ctx->launches;
  return CLOVER_OK;
}

int clover_profile_steps(clover_ctx* ctx, int32_t nsteps, double* ms_out, int64_t* launches_out,
                         int32_t nslots) {
  if (!ctx || !ms_out || !launches_out || nslots < NPROF || nsteps < 0)
    return fail(CLOVER_ERR_ARG, "bad arguments");
  for (int i = 0; i < NPROF; ++i) { ms_out[i] = 0.0; launches_out[i] = 0; }
  int rc = join_in(ctx);
  if (rc) return rc;
  rc = ensure_state_rows(ctx);
  ctx->prof = true;
  for (int s = 0; s < nsteps && !rc; ++s) {
    rc = enqueue_step(ctx, ctx->advect_x, 7);
    ctx->state_rows = step_state_rows(ctx);
    ctx->advect_x = !ctx->advect_x;
  }
  ctx->prof = false;
  cudaError_t e = cudaStreamSynchronize(ctx->work);
  for (size_t i = 1; i < ctx->prof_events.size(); ++i) {
    int id = ctx->prof_events[i].first;
    if (id < 0) continue;
    float ms = 0.f;
    cudaEventElapsedTime(&ms, ctx->prof_events[i - 1].second, ctx->prof_events[i].second);
    ms_out[id & (PROF_FIXUP - 1)] += ms;
    if (!(id & PROF_FIXUP)) launches_out[id] += 1;
  }
  for (auto& pe : ctx->prof_events) cudaEventDestroy(pe.second);
  ctx->prof_events.clear();
  if (rc) return rc;
  if (e != cudaSuccess) return fail(CLOVER_ERR_CUDA, cudaGetErrorString(e));
  rc = check_err(ctx);
  if (rc) return rc;
  return join_out(ctx);
}

// Self-check of div_rn (clover_common.cuh) against IEEE a/b on random
// operands: exponents in [-emax, emax], random signs and mantissas, one
// numerator in 16 is +-0.  Counts bitwise mismatches.
__device__ __forceinline__ unsigned long long splitmix(unsigned long long x) {
  x += 0x9E3779B97F4A7C15ull;
  x = (x ^ (x >> 30)) * 0xBF58476D1CE4E5B9ull;
  x = (x ^ (x >> 27)) * 0x94D049BB133111EBull;
  return x ^ (x >> 31);
}
__device__ __forceinline__ double rand_double(unsigned long long r, int emin, int emax) {
  const unsigned long long mant = r & 0xFFFFFFFFFFFFFull;
  const int e = (int)((r >> 52) % (unsigned long long)(emax - emin + 1)) + emin;
  const unsigned long long sign = (r >> 63) << 63;
  const unsigned long long bits = sign | ((unsigned long long)(1023 + e) << 52) | mant;
  return __longlong_as_double((long long)bits);
}
__global__ void k_div_check(long long n, unsigned long long seed, int emax,
                            unsigned long long* bad, double* example) {
  for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n;
       i += (long long)gridDim.x * blockDim.x) {
    const unsigned long long r1 = splitmix(seed ^ (2 * i)), r2 = splitmix(seed ^ (2 * i + 1));
    // contract of DivFast (clover_common.cuh): divisor in [2^-900, 2^900]
    // (here [2^-300, 2^300]), quotient below 2^900; numerators anywhere
    // down to denormals and zero.
    double a = rand_double(r1, -emax, emax < 600 ? emax : 600);
    double b = rand_double(r2 >> 1, -(emax < 300 ? emax : 300), emax < 300 ? emax : 300);
    if ((r2 & 15) == 0) a = (r1 & 1) ? -0.0 : 0.0;
    clover::DivFast f;
    double q1 = f(a, b);
    if (f.bad) q1 = a / b;
    const double q2 = a / b;
    // constant-divisor form with the correctly rounded reciprocal
    clover::DivFast fc;
    const double rb = 1.0 / b;
    double q3 = fc.c(a, b, rb);
    if (fc.bad) q3 = a / b;
    if (__double_as_longlong(q1) != __double_as_longlong(q2) ||
        __double_as_longlong(q3) != __double_as_longlong(q2)) {
      if (atomicAdd(bad, 1ull) == 0) { example[0] = a; example[1] = b; }
    }
  }
}

int clover_debug_div_check(int64_t n, uint64_t seed, int32_t emax, int64_t* mismatches,
                           double* example_ab) {
  if (!mismatches || n < 0 || emax < 1 || emax > 1023) return fail(CLOVER_ERR_ARG, "bad arguments");
  unsigned long long* d_bad = nullptr;
  double* d_ex = nullptr;
  CK(cudaMalloc(&d_bad, sizeof(unsigned long long)));
  CK(cudaMalloc(&d_ex, 2 * sizeof(double)));
  CK(cudaMemset(d_bad, 0, sizeof(unsigned long long)));
  CK(cudaMemset(d_ex, 0, 2 * sizeof(double)));
  k_div_check<<<148 * 16, 256>>>(n, seed, emax, d_bad, d_ex);
  CK(cudaGetLastError());
  unsigned long long h = 0;
  double ex[2] = {0, 0};
  CK(cudaMemcpy(&h, d_bad, sizeof(h), cudaMemcpyDeviceToHost));
  CK(cudaMemcpy(ex, d_ex, sizeof(ex), cudaMemcpyDeviceToHost));
  cudaFree(d_bad);
  cudaFree(d_ex);
  *mismatches = (int64_t)h;
  if (example_ab) { example_ab[0] = ex[0]; example_ab[1] = ex[1]; }
  return CLOVER_OK;
}

const char* clover_profile_name(int32_t i) { return (i >= 0 && i < NPROF) ? kProfNames[i] : ""; }

int clover_debug_partial_step(clover_ctx* ctx, int32_t nkernels) {
  if (!ctx) return fail(CLOVER_ERR_ARG, "ctx is NULL");
  int rc = join_in(ctx);
  if (rc) return rc;
  rc = ensure_state_rows(ctx);
  if (!rc) rc = enqueue_step(ctx, ctx->advect_x, nkernels);
  if (rc) return rc;
  if (nkernels >= 6) ctx->state_rows = step_state_rows(ctx);  // sweep 2 rewrote the state
  return join_out(ctx);
}

int clover_sync(clover_ctx* ctx) {
  if (!ctx) return fail(CLOVER_ERR_ARG, "ctx is NULL");
  return check_err(ctx);
}

int clover_get_clock(clover_ctx* ctx, int32_t* step, double* time, double* dt_last) {
  if (!ctx) return fail(CLOVER_ERR_ARG, "ctx is NULL");
  int rc = check_err(ctx);
  StepScalars h;
  CK(cudaMemcpy(&h, ctx->scal, sizeof(h), cudaMemcpyDeviceToHost));
  if (step) *step = h.step;
  if (time) *time = h.time;
  if (dt_last) *dt_last = h.dt;
  return rc;
}

int clover_dt_history(clover_ctx* ctx, int32_t first, int32_t n, double* host_out) {
  if (!ctx || !host_out || n < 0 || first < 1) return fail(CLOVER_ERR_ARG, "bad arguments");
  CK(cudaStreamSynchronize(ctx->work));
  StepScalars h;
  CK(cudaMemcpy(&h, ctx->scal, sizeof(h), cudaMemcpyDeviceToHost));
  if (first + n - 1 > h.step || h.step - first >= DT_HIST) return fail(CLOVER_ERR_ARG, "steps outside the kept history");
  if (n > 0 && first < ctx->hist_first)
    return fail(CLOVER_ERR_ARG, "steps before the restart point are not in the history");
  std::vector<double> all(DT_HIST);
  CK(cudaMemcpy(all.data(), ctx->hist, DT_HIST * 8, cudaMemcpyDeviceToHost));
  for (int i = 0; i < n; ++i) host_out[i] = all[(first - 1 + i) % DT_HIST];
  return CLOVER_OK;
}

int clover_field_summary(clover_ctx* ctx, clover_summary* out) {
  if (!ctx || !out) return fail(CLOVER_ERR_ARG, "NULL argument");
  int rc = join_in(ctx);
  if (rc) return rc;
  for (auto& cs : ctx->chunks) {
    k_summary<<<dim3(cs.ntx, cs.nty), dim3(ST, ST), 0, ctx->work>>>(
        cs.c, cs.buf[B_D0], cs.buf[B_E0], cs.buf[B_U0], cs.buf[B_V0], cs.partials);
    LAUNCH_CHECK();
  }
  // tile partials of every chunk of the mesh, in chunk-id order (all ranks'
  // chunks after an all-gather of the padded per-rank blocks)
  const int nch = ctx->L.px * ctx->L.py;
  auto ntiles = [&](int id) {
    const int cx = id % ctx->L.px, cy = id / ctx->L.px;
    const int nx = ctx->L.xs[cx + 1] - ctx->L.xs[cx], ny = ctx->L.ys[cy + 1] - ctx->L.ys[cy];
    return std::make_pair((nx + ST - 1) / ST, (ny + ST - 1) / ST);
  };
  std::vector<std::vector<double>> per(nch);
  if (ctx->nranks == 1) {
    for (auto& cs : ctx->chunks) {
      per[cs.id].resize((size_t)cs.ntx * cs.nty * 5);
      CK(cudaMemcpyAsync(per[cs.id].data(), cs.partials, per[cs.id].size() * 8, cudaMemcpyDeviceToHost,
                         ctx->work));
    }
    rc = check_err(ctx);
  } else {
    int64_t maxt = 0;
    for (int id = 0; id < nch; ++id) {
      auto t = ntiles(id);
      maxt = std::max<int64_t>(maxt, (int64_t)t.first * t.second * 5);
    }
    const int64_t cnt = (int64_t)ctx->chunks.size() * maxt;
    double* pack = nullptr;
    CK(cudaMallocAsync((void**)&pack, (size_t)cnt * 8, ctx->work));
    for (size_t t = 0; t < ctx->chunks.size(); ++t) {
      auto& cs = ctx->chunks[t];
      CK(cudaMemcpyAsync(pack + t * maxt, cs.partials, (size_t)cs.ntx * cs.nty * 5 * 8,
                         cudaMemcpyDeviceToDevice, ctx->work));
    }
    std::vector<double> all((size_t)cnt * ctx->nranks);
    rc = allgather_to_host(ctx, pack, cnt, all.data());
    cudaFreeAsync(pack, ctx->work);
    if (rc) return rc;
    for (int r = 0; r < ctx->nranks; ++r) {
      const std::vector<int> ids = local_chunk_ids(ctx->L.px, ctx->L.py, r, ctx->nranks);
      for (size_t t = 0; t < ids.size(); ++t) {
        auto nt = ntiles(ids[t]);
        const double* blk = all.data() + (size_t)r * cnt + t * maxt;
        per[ids[t]].assign(blk, blk + (size_t)nt.first * nt.second * 5);
      }
    }
    rc = check_err(ctx);
  }
  double acc[5] = {0, 0, 0, 0, 0};
  if (ctx->L.tile_aligned) {
    // 16x16 tiles aligned at global cell 1: sum in global tile order, so
    // every decomposition (chunks, ranks) gives the same bits
    const int GTX = (ctx->g.x_cells + ST - 1) / ST, GTY = (ctx->g.y_cells + ST - 1) / ST;
    std::vector<double> glob((size_t)GTX * GTY * 5, 0.0);
    for (int id = 0; id < nch; ++id) {
      auto nt = ntiles(id);
      const int tx0 = ctx->L.xs[id % ctx->L.px] / ST, ty0 = ctx->L.ys[id / ctx->L.px] / ST;
      for (int ty = 0; ty < nt.second; ++ty)
        for (int tx = 0; tx < nt.first; ++tx)
          for (int q = 0; q < 5; ++q)
            glob[((size_t)(ty0 + ty) * GTX + (tx0 + tx)) * 5 + q] = per[id][((size_t)ty * nt.first + tx) * 5 + q];
    }
    for (size_t t = 0; t < (size_t)GTX * GTY; ++t)
      for (int q = 0; q < 5; ++q) acc[q] = acc[q] + glob[t * 5 + q];
  } else {
    for (auto& v : per)
      for (size_t t = 0; t < v.size() / 5; ++t)
        for (int q = 0; q < 5; ++q) acc[q] = acc[q] + v[t * 5 + q];
  }
  out->vol = acc[0]; out->mass = acc[1]; out->ie = acc[2]; out->ke = acc[3]; out->press = acc[4];
  int rc2 = join_out(ctx);
  if (!rc && (std::isnan(acc[0]) || std::isnan(acc[1]) || std::isnan(acc[2]) || std::isnan(acc[3]) ||
              std::isnan(acc[4])))
    rc = fail(CLOVER_ERR_NAN, "field_summary: a total is NaN");
  return rc ? rc : rc2;
}

int clover_read_field(clover_ctx* ctx, int32_t field_id, double* host, int64_t n) {
  if (!ctx || !host) return fail(CLOVER_ERR_ARG, "NULL argument");
  FieldMap m;
  if (field_map(field_id, &m)) return fail(CLOVER_ERR_ARG, "unknown field id");
  int rc = join_in(ctx);
  if (rc) return rc;
  if (field_id == CLOVER_F_PRESSURE || field_id == CLOVER_F_SOUNDSPEED) {
    for (auto& cs : ctx->chunks) {
      k_eos_field<<<cell_grid(cs.c, 32, 8), dim3(32, 8), 0, ctx->work>>>(
          cs.c, cs.buf[B_D0], cs.buf[B_E0], cs.buf[B_SCR], field_id == CLOVER_F_SOUNDSPEED);
      LAUNCH_CHECK();
    }
  }
  rc = gather_all(ctx, m.buf, kBufKind[m.buf], host, n);
  if (rc) return rc;
  return check_err(ctx);
}

int clover_read_field_window(clover_ctx* ctx, int32_t field_id, int32_t j0, int32_t k0, int32_t w,
                             int32_t h, double* host) {
  if (!ctx || !host) return fail(CLOVER_ERR_ARG, "NULL argument");
  if (ctx->nranks > 1) return fail(CLOVER_ERR_STATE, "windowed read is single-process only");
  FieldMap m;
  if (field_map(field_id, &m)) return fail(CLOVER_ERR_ARG, "unknown field id");
  int ax, ay;
  const int kind = kBufKind[m.buf];
  kind_extra(kind, &ax, &ay);
  const int NXE = ctx->g.x_cells + ax, NYE = ctx->g.y_cells + ay;
  if (w < 1 || h < 1 || j0 < 1 || k0 < 1 || j0 + w - 1 > NXE || k0 + h - 1 > NYE)
    return fail(CLOVER_ERR_ARG, "window outside the field's global interior");
  int rc = join_in(ctx);
  if (rc) return rc;
  if (field_id == CLOVER_F_PRESSURE || field_id == CLOVER_F_SOUNDSPEED) {
    for (auto& cs : ctx->chunks) {
      k_eos_field<<<cell_grid(cs.c, 32, 8), dim3(32, 8), 0, ctx->work>>>(
          cs.c, cs.buf[B_D0], cs.buf[B_E0], cs.buf[B_SCR], field_id == CLOVER_F_SOUNDSPEED);
      LAUNCH_CHECK();
    }
  }
  for (auto& cs : ctx->chunks) {
    const Chunk& c = cs.c;
    // owned global range of this chunk for the kind (shared last node/face
    // only on the global edge), intersected with the window
    const int cw = c.nx + ((c.gj0 + c.nx == ctx->g.x_cells) ? ax : 0);
    const int ch = c.ny + ((c.gk0 + c.ny == ctx->g.y_cells) ? ay : 0);
    const int ja = std::max(j0, c.gj0 + 1), jb = std::min(j0 + w - 1, c.gj0 + cw);
    const int ka = std::max(k0, c.gk0 + 1), kb = std::min(k0 + h - 1, c.gk0 + ch);
    if (ja > jb || ka > kb) continue;
    double* dst = host + (int64_t)(ka - k0) * w + (ja - j0);
    const double* src = cs.buf[m.buf] + idx(c, ja - c.gj0, ka - c.gk0);
    CK(cudaMemcpy2DAsync(dst, (size_t)w * 8, src, (size_t)c.pitch * 8, (size_t)(jb - ja + 1) * 8,
                         kb - ka + 1, cudaMemcpyDeviceToHost, ctx->work));
  }
  return check_err(ctx);
}

int clover_debug_read_buffer(clover_ctx* ctx, int32_t buffer_id, int32_t kind, double* host, int64_t n) {
  if (!ctx || !host) return fail(CLOVER_ERR_ARG, "NULL argument");
  if (buffer_id < 0 || buffer_id >= NBUF) return fail(CLOVER_ERR_ARG, "bad buffer id");
  if (kind < 0 || kind > 4) return fail(CLOVER_ERR_ARG, "bad kind");
  if (ctx->nranks > 1) return fail(CLOVER_ERR_STATE, "multi-rank debug read not supported");
  int rc = join_in(ctx);
  if (rc) return rc;
  return gather_local(ctx, buffer_id, kind, host, n);
}

int clover_write_field(clover_ctx* ctx, int32_t field_id, const double* host, int64_t n) {
  if (!ctx || !host) return fail(CLOVER_ERR_ARG, "NULL argument");
  int buf;
  switch (field_id) {
    case CLOVER_F_DENSITY0: buf = B_D0; break;
    case CLOVER_F_ENERGY0: buf = B_E0; break;
    case CLOVER_F_XVEL0: buf = B_U0; break;
    case CLOVER_F_YVEL0: buf = B_V0; break;
    default: return fail(CLOVER_ERR_ARG, "only density0, energy0, xvel0, yvel0 are writable");
  }
  int rc = join_in(ctx);
  if (rc) return rc;
  rc = scatter_local(ctx, buf, kBufKind[buf], host, n);
  if (rc) return rc;
  rc = reflect_all(ctx, {buf});
  if (rc) return rc;
  CK(cudaStreamSynchronize(ctx->work));
  return join_out(ctx);
}

int clover_step_host(clover_ctx* ctx, int32_t nsteps, const double* d_in, const double* e_in,
                     const double* u_in, const double* v_in, double* d_out, double* e_out,
                     double* u_out, double* v_out) {
  if (!ctx) return fail(CLOVER_ERR_ARG, "ctx is NULL");
  const int64_t nc = (int64_t)ctx->g.x_cells * ctx->g.y_cells;
  const int64_t nn = (int64_t)(ctx->g.x_cells + 1) * (ctx->g.y_cells + 1);
  int rc = join_in(ctx);
  if (rc) return rc;
  const double* ins[4] = {d_in, e_in, u_in, v_in};
  const int bufs[4] = {B_D0, B_E0, B_U0, B_V0};
  for (int f = 0; f < 4; ++f)
    if (ins[f]) {
      rc = scatter_local(ctx, bufs[f], kBufKind[bufs[f]], ins[f], f < 2 ? nc : nn);
      if (rc) return rc;
    }
  rc = reflect_all(ctx, {B_D0, B_E0, B_U0, B_V0});
  if (rc) return rc;
  rc = join_out(ctx);
  if (rc) return rc;
  rc = clover_step(ctx, nsteps);
  if (rc) return rc;
  rc = join_in(ctx);
  if (rc) return rc;
  double* outs[4] = {d_out, e_out, u_out, v_out};
  for (int f = 0; f < 4; ++f)
    if (outs[f]) {
      rc = gather_local(ctx, bufs[f], kBufKind[bufs[f]], outs[f], f < 2 ? nc : nn);
      if (rc) return rc;
    }
  return check_err(ctx);
}

int clover_checkpoint_plan(int32_t loop, uint32_t* save_mask, int32_t* nsaved, const char** name) {
  if (loop < 0 || loop >= kNumLoops) return fail(CLOVER_ERR_ARG, "loop index out of range");
  const unsigned m = checkpoint_plan(loop);
  if (save_mask) *save_mask = m;
  if (nsaved) *nsaved = __builtin_popcount(m);
  if (name) *name = kStepLoops[loop].name;
  return CLOVER_OK;
}

int clover_checkpoint_bytes(clover_ctx* ctx, int64_t* bytes) {
  if (!ctx || !bytes) return fail(CLOVER_ERR_ARG, "NULL argument");
  const int64_t nc = (int64_t)ctx->g.x_cells * ctx->g.y_cells;
  const int64_t nn = (int64_t)(ctx->g.x_cells + 1) * (ctx->g.y_cells + 1);
  *bytes = (int64_t)sizeof(CkptHeader) + 8 * (2 * nc + 2 * nn);
  return CLOVER_OK;
}

int clover_checkpoint(clover_ctx* ctx, void* host, int64_t bytes) {
  if (!ctx || !host) return fail(CLOVER_ERR_ARG, "NULL argument");
  int64_t need;
  clover_checkpoint_bytes(ctx, &need);
  if (bytes < need) return fail(CLOVER_ERR_ARG, "checkpoint buffer too small");
  // the step boundary is the optimum of the access analysis: exactly the
  // four state fields are live there
  if (checkpoint_plan(0) != ((1u << D_RHO0) | (1u << D_E0) | (1u << D_U0) | (1u << D_V0)))
    return fail(CLOVER_ERR_STATE, "checkpoint plan mismatch");
  int rc = join_in(ctx);
  if (rc) return rc;
  rc = check_err(ctx);
  if (rc) return rc;
  StepScalars h;
  CK(cudaMemcpy(&h, ctx->scal, sizeof(h), cudaMemcpyDeviceToHost));
  CkptHeader hd{};
  hd.magic = kCkptMagic; hd.version = 1;
  hd.x_cells = ctx->g.x_cells; hd.y_cells = ctx->g.y_cells; hd.face_mirror = ctx->g.face_mirror;
  hd.step = h.step; hd.advect_x = ctx->advect_x ? 1 : 0; hd.nfields = 4;
  hd.xmin = ctx->g.xmin; hd.ymin = ctx->g.ymin; hd.xmax = ctx->g.xmax; hd.ymax = ctx->g.ymax;
  hd.time = h.time; hd.dt = h.dt; hd.dtold = h.dtold;
  std::memcpy(host, &hd, sizeof(hd));
  double* p = (double*)((char*)host + sizeof(hd));
  const int64_t nc = (int64_t)ctx->g.x_cells * ctx->g.y_cells;
  const int64_t nn = (int64_t)(ctx->g.x_cells + 1) * (ctx->g.y_cells + 1);
  rc = gather_all(ctx, B_D0, K_CELL, p, nc);
  if (!rc) rc = gather_all(ctx, B_E0, K_CELL, p + nc, nc);
  if (!rc) rc = gather_all(ctx, B_U0, K_XVEL, p + 2 * nc, nn);
  if (!rc) rc = gather_all(ctx, B_V0, K_YVEL, p + 2 * nc + nn, nn);
  if (rc) return rc;
  return join_out(ctx);
}

int clover_restart(clover_ctx* ctx, const void* host, int64_t bytes) {
  if (!ctx || !host) return fail(CLOVER_ERR_ARG, "NULL argument");
  int64_t need;
  clover_checkpoint_bytes(ctx, &need);
  if (bytes < need) return fail(CLOVER_ERR_ARG, "checkpoint buffer too small");
  CkptHeader hd;
  std::memcpy(&hd, host, sizeof(hd));
  if (hd.magic != kCkptMagic || hd.version != 1 || hd.nfields != 4)
    return fail(CLOVER_ERR_ARG, "not a clover checkpoint");
  if (hd.x_cells != ctx->g.x_cells || hd.y_cells != ctx->g.y_cells || hd.xmin != ctx->g.xmin ||
      hd.ymin != ctx->g.ymin || hd.xmax != ctx->g.xmax || hd.ymax != ctx->g.ymax ||
      hd.face_mirror != ctx->g.face_mirror)
    return fail(CLOVER_ERR_ARG, "checkpoint was taken on a different mesh");
  const double* p = (const double*)((const char*)host + sizeof(hd));
  const int64_t nc = (int64_t)ctx->g.x_cells * ctx->g.y_cells;
  const int64_t nn = (int64_t)(ctx->g.x_cells + 1) * (ctx->g.y_cells + 1);
  int rc = join_in(ctx);
  if (rc) return rc;
  rc = scatter_local(ctx, B_D0, K_CELL, p, nc);
  if (!rc) rc = scatter_local(ctx, B_E0, K_CELL, p + nc, nc);
  if (!rc) rc = scatter_local(ctx, B_U0, K_XVEL, p + 2 * nc, nn);
  if (!rc) rc = scatter_local(ctx, B_V0, K_YVEL, p + 2 * nc + nn, nn);
  if (rc) return rc;
  rc = reflect_all(ctx, {B_D0, B_E0, B_U0, B_V0});
  if (rc) return rc;
  StepScalars h;
  CK(cudaStreamSynchronize(ctx->work));
  CK(cudaMemcpy(&h, ctx->scal, sizeof(h), cudaMemcpyDeviceToHost));
  h.step = hd.step; h.time = hd.time; h.dt = hd.dt; h.dtold = hd.dtold; h.err = 0;
  ctx->hist_first = hd.step + 1;
  {
    double big = G_BIG;
    std::memcpy(&h.dt_slot, &big, 8);
  }
  CK(cudaMemcpyAsync(ctx->scal, &h, sizeof(h), cudaMemcpyHostToDevice, ctx->work));
  ctx->advect_x = hd.advect_x != 0;
  CK(cudaStreamSynchronize(ctx->work));
  return join_out(ctx);
}

int clover_finalize(clover_ctx* ctx) {
  if (!ctx) return CLOVER_OK;
  int rc = CLOVER_OK;
  if (ctx->work) {
    rc = check_err(ctx);
  }
  for (int i = 0; i < 4; ++i)
    if (ctx->gexec[i]) cudaGraphExecDestroy(ctx->gexec[i]);
  lsa_teardown(ctx);
#ifdef CLOVER_WITH_NCCL
  if (ctx->comm) ncclCommDestroy(ctx->comm);
#endif
  if (ctx->ev_in) cudaEventDestroy(ctx->ev_in);
  if (ctx->ev_b) cudaEventDestroy(ctx->ev_b);
  if (ctx->ev_x) cudaEventDestroy(ctx->ev_x);
  if (ctx->comm_stream) cudaStreamDestroy(ctx->comm_stream);
  if (ctx->ev_out) cudaEventDestroy(ctx->ev_out);
  if (ctx->work) cudaStreamDestroy(ctx->work);
  delete ctx;
  return rc;
}

}  // extern "C"
