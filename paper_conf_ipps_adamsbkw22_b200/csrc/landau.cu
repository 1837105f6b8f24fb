// landau.cu -- liblandau.so: the handle, the launch sequence of one build and the C ABI of
// include/landau.h.  The sm_100a kernels live in
//   kernels.cuh        FP64 pair body (cancellation-free U^D, U^K), coefficients, rcp/rsqrt/log
//   kernels_inner.cuh  a-2: inner_sym_kernel (unordered pairs) / inner_kernel (ordered, split-j),
//                      reduce_sym_kernel / reduce_kernel, tensor_fill_kernel (tensor cache)
//   kernels_fe.cuh     a-1 field_kernel, a-4 element_kernel, a-3 + a-5 assemble_kernel, a-6 mass kernels
//   dynload.h          NCCL (element split) and cuBLAS (tensor cache), loaded on demand
// Citations: see include/landau.h and DESIGN.md.
#include <cuda_runtime.h>
#include <dlfcn.h>

#include <algorithm>
#include <cmath>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <mutex>
#include <string>
#include <vector>

#include "../../include/landau.h"
#include "host_setup.h"
#include "kernels.cuh"

using namespace landau;

#include "dynload.h"
#include "kernels_fe.cuh"
#include "kernels_inner.cuh"
#include "kernels_band.cuh"
#include "kernels_band_mma.cuh"
#include "kernels_single.cuh"
#include "kernels_3d.cuh"
#include "kernels_3d_fe.cuh"


// ==================================================================================================
// handle
// ==================================================================================================
struct landau_s {
  int device = 0;
  cudaStream_t stream = nullptr;
  Plan plan;
  int S = 0;
  std::vector<double> mass, charge;
  std::vector<int> sgrid;
  double nu = 1.0;
  SpeciesConst spc{};
  int64_t ndof = 0, nnz = 0, ncoo = 0;
  std::vector<int64_t> soff, snnz_off, scoo_off;
  // distribution
  int rank = 0, world = 1, mode = 0;
  int64_t e0 = 0, e1 = 0, chunk_cells = 0, Nc = 0;
  ncclComm_ comm = nullptr;
  // device: static
  double *d_r = nullptr, *d_z = nullptr, *d_w = nullptr, *d_h = nullptr, *d_tab = nullptr;
  int *d_cell_grid = nullptr;
  int32_t *d_ext_ptr = nullptr, *d_ext_dof = nullptr;
  double *d_ext_w = nullptr;
  struct DevMap {
    int64_t *ptr = nullptr;
    int32_t *idx = nullptr;
    double *w = nullptr;
    int64_t nslots = 0;
  };
  std::vector<DevMap> d_csr, d_coo;
  GatherDev *d_gmaps[2] = {nullptr, nullptr};   // per format (CSR, COO): the grids' gather maps (tail_kernel)
  // tail_kernel (fused a-4 + a-5) phased gather maps per format; tail_ok: built and fit shared memory
  struct TailMaps {
    int32_t *grid_phase_ptr = nullptr, *cell_ptr = nullptr, *slot_ptr = nullptr, *meta = nullptr, *idx4 = nullptr,
            *optr = nullptr, *oidx = nullptr;
    double *w4 = nullptr, *ow = nullptr;
    int max_cells = 0, max_cross = 0, nphases = 0;
  } tmaps[2];
  bool tail_ok = false;
  size_t tail_smem = 0;
  std::vector<double *> d_mass_csr, d_mass_coo;   // per grid
  std::vector<double *> d_adv_csr, d_adv_coo;     // per grid: unscaled E_z advection matrix (NEXT-3)
  std::vector<int64_t *> d_rowptr;                // per grid: CSR pattern of one species block
  std::vector<int32_t *> d_col;
  // implicit step (NEXT-3) workspace
  double *d_Jwork = nullptr, *d_rhs = nullptr, *d_norms = nullptr, *h_norms = nullptr;
  double *d_srcx = nullptr;   // f_old / dt + sigma (implicit step with a source)
  int64_t step_cap = 0;
  // device: state + workspace
  int64_t cap = 0, nbatch = 0, chunk = 1;
  bool have_state = false;
  double *d_f = nullptr, *d_wT = nullptr, *d_part = nullptr, *d_G = nullptr, *d_C = nullptr;
  int64_t part_cap = 0;
  SymItem *d_sym_items = nullptr;   // work items of the symmetric inner kernel
  int32_t *d_tile_ptr = nullptr, *d_tile_slots = nullptr;
  int ntiles = 0;
  int64_t nsym_items = 0, nsym_slots = 0;
  // mirror-symmetric inner kernel (meshes symmetric under z -> -z): upper-half points u, their
  // original indices pu and mirrors pm, work items and slot map over the tiles of the upper half
  bool mirror_sym = false; // every grid's points pair up bit-exactly under z -> -z (detect_mirror)
  std::vector<int32_t> mir_pu, mir_pm;   // host copies of the pairing (upper half, mirror)
  bool mirror = false;     // the mirror kernels are set up (maps built on the device)
  bool dist_pairs = false; // element-split mode on a mirror mesh: tile pairs split over ranks + all-reduce
  int64_t mir_evals = 0;   // tensor evaluations per batch item of this handle's slot-kernel items
  bool mirror_on = true;   // use inner_mir_kernel when the symmetric path runs (landau_set_mirror)
  int mirror_mode = 1;     // 1: auto (per-vertex kernel for large batches), 2: slot kernel, 3: per-vertex kernel
  int64_t H = 0;
  // per-vertex mirror kernel (inner_vtx_kernel): round schedule of tile-pair items
  VtxItem *d_vtx_items = nullptr;
  int32_t *d_vtx_round_ptr = nullptr;
  int nvtx_rounds = 0;
  size_t vtx_smem = 0;     // dynamic shared memory (Ga, Gb); 0 when the vertex does not fit
  int32_t *d_vtx_wp = nullptr;       // stream-K: prefix of the round weights [nrounds + 1]
  std::vector<int32_t> vtx_w;        // the rounds' weights (canonical order)
  // per-batch stream-K tables (vtx_tables): round order and weight prefix per vertex, for (nbatch, S)
  int16_t *d_vtx_ord = nullptr;
  int32_t *d_vtx_wpv = nullptr;
  int64_t vtx_tab_nb = -1;
  int vtx_tab_S = -1;
  int64_t vtx_Wv = 0;                // weight of one vertex
  double *d_vtx_part = nullptr;      // stream-K partial slots [grid][2][10 Hp]
  int32_t *d_vtx_cnt = nullptr;      // stream-K per-vertex arrival counters [cap] (zero between builds)
  int64_t vtx_cnt_cap = 0;
  double *d_rU = nullptr, *d_zU = nullptr;
  int32_t *d_pu = nullptr, *d_pm = nullptr;
  int32_t *d_pinv = nullptr;   // point -> upper-half index (+ H for a mirror point): the fused build's a-4
  // slot-kernel item sets: [0] one i-tile per item (fine-grained: small batches), [1] runs of up to
  // LANDAU_MIR_RUN i-tiles per j-tile (fewer slots and stagings: large work, e.g. C5)
  struct MirSet {
    int4 *items = nullptr;
    int32_t *tile_ptr = nullptr, *tile_slots = nullptr;
    int64_t nitems = 0, nslots = 0;
  } mset[2];
  bool coincident = false;   // two distinct quadrature points with identical (r, z) (never for one grid)
  // tensor cache (NEXT-4)
  bool tcache = false, tcache_valid = false;
  bool tcache_recompute = false;   // landau_set_tensor_cache(h, 2): evaluate the tensors in every build
  double *d_U = nullptr;     // A1 (3N^2) | A2 (2N^2) | A3 (2N^2)
  cublasHandle_ cublas = nullptr;
  // band solver (NEXT-2)
  std::vector<int32_t *> d_ent_ptr, d_ent_slot;   // per grid: entering-row entry lists (host_setup.h)
  std::vector<uint16_t *> d_ent_pos;
  int band_ent_max = 0;
  int64_t ent_bstride = 0;
  double *d_Aent = nullptr;
  BandDesc *d_band_desc = nullptr;      // per species
  std::vector<BandDesc> band_desc;
  int32_t *d_perm_all = nullptr;
  int64_t *d_perm_off = nullptr, *d_vec_off = nullptr;
  int64_t band_bstride = 0, band_cap = 0, band_nbatch = 0;
  double *d_band = nullptr;   // step-major LU factors [batch][band_bstride] (kernels_band.cuh)
  double *d_yfwd = nullptr;   // forward-eliminated right-hand side of the fused factorisation [batch][ndof]
  int64_t yfwd_cap = 0;
  bool band_fwd_done = false; // the last factorisation eliminated the rhs and stored U only
  // host staging for landau_jacobian_host: full-batch device buffers, two copy streams
  double *d_vals_tmp = nullptr;
  int64_t vals_tmp_cap = 0;
  cudaStream_t s_h2d = nullptr, s_d2h = nullptr;
  std::vector<cudaEvent_t> ev_h2d, ev_built;
  const double *fin = nullptr;   // state read by the field kernel (nullptr: d_f)
  landau_stats_t stats{};        // how the last build ran
  // timing
  bool timing = false;
  std::vector<std::pair<int, std::pair<cudaEvent_t, cudaEvent_t>>> ev_used;
  std::vector<cudaEvent_t> ev_pool;
  int64_t tlaunch[LANDAU_NTIMERS] = {0};
  int64_t launches = 0;
  bool host_only = false;
  // CUDA graphs of whole builds (no per-stage timers): key (nbatch, format, out) -> exec, kernels
  struct GraphEntry {
    int64_t nbatch;
    int format;
    double *out;
    const double *fin;
    cudaGraphExec_t exec;
    int64_t kernels;
  };
  std::vector<GraphEntry> graphs;
  bool use_graphs = true;
  std::string err;
};

namespace {

int fail(landau_t h, int code, const std::string &msg) {
  if (h) h->err = msg;
  else g_create_error = msg;
  return code;
}

#define CU(call)                                                                                   \
  do {                                                                                             \
    cudaError_t e_ = (call);                                                                       \
    if (e_ != cudaSuccess) return fail(h, LANDAU_ECUDA, std::string(#call) + ": " + cudaGetErrorString(e_)); \
  } while (0)

#define KCHECK()                                                                                   \
  do {                                                                                             \
    cudaError_t e_ = cudaGetLastError();                                                           \
    if (e_ != cudaSuccess) return fail(h, LANDAU_ECUDA, std::string("kernel launch: ") + cudaGetErrorString(e_)); \
  } while (0)

template <class T>
int upload(landau_t h, T **dst, const std::vector<T> &src) {
  size_t bytes = std::max<size_t>(src.size(), 1) * sizeof(T);
  CU(cudaMalloc((void **)dst, bytes));
  if (!src.empty()) CU(cudaMemcpyAsync(*dst, src.data(), src.size() * sizeof(T), cudaMemcpyHostToDevice, h->stream));
  return LANDAU_OK;
}

cudaEvent_t get_event(landau_t h) {
  if (!h->ev_pool.empty()) {
    cudaEvent_t e = h->ev_pool.back();
    h->ev_pool.pop_back();
    return e;
  }
  cudaEvent_t e;
  cudaEventCreate(&e);
  return e;
}

struct Timer {
  landau_t h;
  int stage;
  cudaEvent_t a = nullptr, b = nullptr;
  Timer(landau_t h_, int s) : h(h_), stage(s) {
    if (h->timing) {
      a = get_event(h);
      b = get_event(h);
      cudaEventRecord(a, h->stream);
    }
  }
  ~Timer() {
    if (h->timing) {
      cudaEventRecord(b, h->stream);
      h->ev_used.push_back({stage, {a, b}});
    }
  }
};

void drop_graphs(landau_t h) {
  for (auto &g : h->graphs) cudaGraphExecDestroy(g.exec);
  h->graphs.clear();
}

int ensure_workspace(landau_t h, int64_t nbatch) {
  const int64_t N = h->plan.npts, Ne = h->plan.ncell, nb = h->plan.nb;
  if (nbatch <= h->cap) return LANDAU_OK;
  drop_graphs(h);
  cudaFree(h->d_f);
  cudaFree(h->d_wT);
  cudaFree(h->d_G);
  cudaFree(h->d_C);
  h->d_f = h->d_wT = h->d_G = h->d_C = nullptr;
  CU(cudaMalloc(&h->d_f, sizeof(double) * nbatch * std::max<int64_t>(h->ndof, 1)));
  CU(cudaMalloc(&h->d_wT, sizeof(double) * nbatch * 3 * N));
  CU(cudaMalloc(&h->d_G, sizeof(double) * nbatch * 5 * h->Nc * h->world));
  // element-matrix chunk: <= ~40 MB so the element kernel's output is still in L2 (126 MB) when the
  // assembly gathers it
  const int64_t per = Ne * 2 * nb * nb * (int64_t)sizeof(double);
  static const int64_t chunk_mb = [] {
    const char *e = getenv("LANDAU_CHUNK_MB");
    return e ? (int64_t)atoll(e) : (int64_t)0;   // 0: one chunk (measured fastest on B200)
  }();
  h->chunk = chunk_mb <= 0 ? nbatch : std::max<int64_t>(1, std::min<int64_t>(nbatch, (chunk_mb << 20) / per));
  CU(cudaMalloc(&h->d_C, sizeof(double) * h->chunk * Ne * 2 * nb * nb));
  h->cap = nbatch;
  return LANDAU_OK;
}

// ---------------------------------------------------------------------------------------------
// launch helpers
// ---------------------------------------------------------------------------------------------
int num_sms(landau_t h) {
  static int sms[64] = {0};
  int &s = sms[h->device & 63];
  if (!s) cudaDeviceGetAttribute(&s, cudaDevAttrMultiProcessorCount, h->device);
  return s ? s : 148;
}

template <int NB>
int launch_field(landau_t h, int64_t nbatch) {
  constexpr int EPB = NB == 9 ? 8 : (NB == 16 ? 8 : 4);
  const Plan &P = h->plan;
  const int64_t items = (P.ncell + EPB - 1) / EPB * nbatch;
  static const int64_t blocks_per_sm = [] {   // grid cap (LANDAU_FIELD_BLOCKS_PER_SM)
    const char *e = getenv("LANDAU_FIELD_BLOCKS_PER_SM");
    return e ? (int64_t)atoll(e) : (int64_t)6;   // C4 1024: 8 43.5 us, 6 35.4, 4 41.8; 128: 16.6, 13.9, 13.9
  }();
  // whole multiples of the chunk count: block g * nchunks + c keeps chunk c (see field_kernel)
  const int64_t nchunks = (P.ncell + EPB - 1) / EPB;
  const int64_t G = std::max<int64_t>(1, std::min<int64_t>(nbatch, blocks_per_sm * num_sms(h) / nchunks));
  const unsigned grid = (unsigned)(G * nchunks);
  (void)items;
  Timer t(h, LANDAU_T_FIELD);
  if (nchunks * nbatch < num_sms(h)) {   // small builds (a single C2 grid: 9 blocks): one cell per block
    field_kernel<NB, 1><<<(unsigned)(P.ncell * std::max<int64_t>(1, std::min<int64_t>(nbatch, num_sms(h)))), NB, 0,
                          h->stream>>>(P.ncell, (int)nbatch, h->ndof, h->fin ? h->fin : h->d_f, h->d_ext_ptr,
                                       h->d_ext_dof, h->d_ext_w, h->d_cell_grid, h->d_h, h->d_w, h->d_tab, h->spc,
                                       h->d_wT, P.npts);
  } else {
    field_kernel<NB, EPB><<<grid, NB * EPB, 0, h->stream>>>(P.ncell, (int)nbatch, h->ndof, h->fin ? h->fin : h->d_f,
                                                            h->d_ext_ptr, h->d_ext_dof, h->d_ext_w, h->d_cell_grid,
                                                            h->d_h, h->d_w, h->d_tab, h->spc, h->d_wT, P.npts);
  }
  h->launches++;
  h->tlaunch[LANDAU_T_FIELD]++;
  KCHECK();
  return LANDAU_OK;
}


// N3 + N4 fused into tail_kernel (one CTA per batch item, each phase's element matrices in shared memory)
// for batches of small meshes: all targets on this GPU, at least LANDAU_TAIL_MIN_BATCH items (fewer
// items would leave most SMs idle: the two-kernel form spreads the cells), phases that fit shared
// memory.  Opt-in (LANDAU_TAIL=1): C4 0.43 ms vs 0.30 ms for element_sf_kernel + assemble_kernel -- the
// hanging-node expansion gives some slots up to 36 contributions, serial per thread.
bool use_tail(landau_t h, int64_t nbatch) {
  static const bool on = [] {   // off by default: measured slower than element_sf + assemble
    const char *e = getenv("LANDAU_TAIL");
    return e && atoi(e) != 0;
  }();
  static const int64_t min_batch = [] {
    const char *e = getenv("LANDAU_TAIL_MIN_BATCH");
    return e ? (int64_t)atoll(e) : (int64_t)16;
  }();
  return on && h->tail_ok && h->Nc == h->plan.npts && h->world == 1 && nbatch >= min_batch;
}

int64_t tail_grid(landau_t h, int64_t nbatch) { return std::min<int64_t>(nbatch, num_sms(h)); }

bool fused_single_enabled();
bool fused_single_ok(landau_t h, int64_t nbatch);

struct InnerPlan {
  bool vtx = false;    // mirror-symmetric per-vertex kernel, stream-K over (vertex, round) work
  bool sym;   // symmetric pair evaluation (whole point set as targets, enough tile pairs to fill the GPU)
  bool mdir = false;   // mirror-symmetric directed kernel (single builds / small batches on z-mirror meshes)
  int tpt;
  int64_t wtiles, nsplit, split_len;
};

// minimum (batch x symmetric work items) per SM for the symmetric kernel (LANDAU_SYM_MIN_ITEMS_PER_SM)
int64_t sym_min_items_per_sm() {
  static const int64_t v = [] {
    const char *e = getenv("LANDAU_SYM_MIN_ITEMS_PER_SM");
    return e ? (int64_t)atoll(e) : (int64_t)4 * kSymWarps * LANDAU_SYM_MINB;   // 4 items per resident warp
  }();
  return v;
}

bool sym_enabled() {
  static const bool v = [] {
    const char *e = getenv("LANDAU_SYM");
    return !(e && atoi(e) == 0);
  }();
  return v;
}

// mirror-symmetric inner kernel when the mesh allows it (LANDAU_MIRROR=0 disables)
bool mirror_enabled() {
  static const bool v = [] {
    const char *e = getenv("LANDAU_MIRROR");
    return !(e && atoi(e) == 0);
  }();
  return v;
}

// per-vertex mirror kernel (automatic mode) when the batch gives every SM at least this much round
// weight (a full round of pair items weighs 2; LANDAU_VTX_MIN_WEIGHT_PER_SM)
int64_t vtx_min_weight_per_sm() {
  static const int64_t v = [] {
    const char *e = getenv("LANDAU_VTX_MIN_WEIGHT_PER_SM");
    return e ? (int64_t)atoll(e) : (int64_t)8;
  }();
  return v;
}

// inner-kernel variant (targets per thread, min blocks per SM); LANDAU_INNER_VARIANT overrides
int inner_variant() {
  static const int v = [] {
    const char *e = getenv("LANDAU_INNER_VARIANT");
    return e ? atoi(e) : 1;
  }();
  return v;
}

// Work decomposition of N2 for a batch, and the split-j partial buffer (allocated here, outside any
// graph capture).
int inner_plan(landau_t h, int64_t nbatch, InnerPlan &ip) {
  const Plan &P = h->plan;
  const int64_t N = P.npts, nt = (h->e1 - h->e0) * P.nqp;
  const int variant = inner_variant();
  ip.vtx = h->mirror && h->mirror_on && h->vtx_smem && !h->dist_pairs &&
           (h->mirror_mode == 3 ||
            (h->mirror_mode == 1 && sym_enabled() &&
             nbatch * h->vtx_Wv >= vtx_min_weight_per_sm() * num_sms(h) * kVtxMinB));
  if (ip.vtx) {   // stream-K partial slots (one pair per CTA) and per-vertex arrival counters
    if (!h->d_vtx_part) {
      const int64_t Hp = (h->H + 31) / 32 * 32;
      CU(cudaMalloc(&h->d_vtx_part, sizeof(double) * (int64_t)num_sms(h) * kVtxMinB * 2 * 10 * Hp));
    }
    if (nbatch > h->vtx_cnt_cap) {
      drop_graphs(h);
      cudaFree(h->d_vtx_cnt);
      h->d_vtx_cnt = nullptr;
      CU(cudaMalloc(&h->d_vtx_cnt, sizeof(int32_t) * nbatch));
      CU(cudaMemsetAsync(h->d_vtx_cnt, 0, sizeof(int32_t) * nbatch, h->stream));
      h->vtx_cnt_cap = nbatch;
    }
    ip.sym = false;
    ip.tpt = 1;
    ip.wtiles = (h->H + 31) / 32;
    ip.nsplit = 1;
    ip.split_len = h->H;
    return LANDAU_OK;
  }
  // symmetric path: all targets on this rank (no element split across ranks), enough work items to
  // fill the GPU, and partial slots within 24 GiB (C5: ~11 GiB of the 180 GB HBM)
  ip.sym = sym_enabled() && h->world == 1 && h->nsym_items > 0 && nbatch * h->nsym_items >= sym_min_items_per_sm() * num_sms(h) &&
           nbatch * h->nsym_slots * 160 * (int64_t)sizeof(double) <= (24LL << 30);
  if (h->dist_pairs) ip.sym = true;   // the rank's share of the mirror items (slot kernel)
  if (ip.sym) {
    ip.tpt = 1;
    ip.wtiles = h->ntiles;
    ip.nsplit = 1;
    ip.split_len = N;
    const int64_t need = (h->mirror && h->mirror_on) ? nbatch * std::max(h->mset[0].nslots, h->mset[1].nslots) * 320
                                                     : nbatch * h->nsym_slots * 160;
    if (need > h->part_cap) {
      drop_graphs(h);
      cudaFree(h->d_part);
      h->d_part = nullptr;
      CU(cudaMalloc(&h->d_part, sizeof(double) * need));
      h->part_cap = need;
    }
    return LANDAU_OK;
  }
  static const bool mdir_on = [] {
    const char *e = getenv("LANDAU_MDIR");
    return !(e && atoi(e) == 0);
  }();
  if (mdir_on && h->mirror && h->mirror_on) {   // targets and sources: the H upper-half points
    const int64_t T = (h->H + 31) / 32;
    ip.mdir = true;
    ip.tpt = 1;
    ip.wtiles = T;
    static const int64_t mdir_wps = [] {   // warps per SM to aim for, minimum sources per split
      const char *e = getenv("LANDAU_MDIR_WARPS_PER_SM");
      return e ? (int64_t)atoll(e) : (int64_t)12;
    }();
    static const int64_t mdir_min = [] {
      const char *e = getenv("LANDAU_MDIR_SPLIT_MIN");
      return e ? (int64_t)atoll(e) : (int64_t)16;   // measured: 16 best on C2/C3 (finer splits cost reduction time)
    }();
    // the fused single-build kernel wants one CTA item (a target tile and a group of 8 source splits)
    // per SM; the stand-alone kernel LANDAU_MDIR_WARPS_PER_SM warps per SM with >= 16 sources per split
    const bool fused = fused_single_ok(h, nbatch);
    int64_t nsplit;
    if (fused) {   // fused kernel: groups of 8 splits per CTA, one CTA item per SM, splits >= 8 sources
      const int64_t ngroups = std::max<int64_t>(1, num_sms(h) / (T * nbatch));
      nsplit = std::min<int64_t>(ngroups * kSbWarps, std::max<int64_t>(1, h->H / 8));
    } else {
      const int64_t want = mdir_wps * num_sms(h);
      nsplit = std::max<int64_t>(1, (want + T * nbatch - 1) / (T * nbatch));
      nsplit = std::min<int64_t>(nsplit, std::max<int64_t>(1, h->H / mdir_min));
    }
    ip.split_len = (h->H + nsplit - 1) / nsplit;
    ip.nsplit = (h->H + ip.split_len - 1) / ip.split_len;
    if (ip.nsplit > 1) {
      const int64_t need = nbatch * ip.nsplit * 10 * T * 32;
      if (need > h->part_cap) {
        drop_graphs(h);
        cudaFree(h->d_part);
        h->d_part = nullptr;
        CU(cudaMalloc(&h->d_part, sizeof(double) * need));
        h->part_cap = need;
      }
    }
    return LANDAU_OK;
  }
  ip.tpt = variant == 0 ? 1 : (variant == 4 ? 4 : 2);
  ip.wtiles = (nt + 32 * ip.tpt - 1) / (32 * ip.tpt);
  // split-j so that small problems still fill the machine: aim for >= LANDAU_SPLIT_WARPS_PER_SM
  // warps per SM, splits of at least LANDAU_SPLIT_MIN sources
  static const int64_t split_wps = [] {
    const char *e = getenv("LANDAU_SPLIT_WARPS_PER_SM");
    return e ? (int64_t)atoll(e) : (int64_t)12;
  }();
  static const int64_t split_min = [] {
    const char *e = getenv("LANDAU_SPLIT_MIN");
    return e ? (int64_t)atoll(e) : (int64_t)32;
  }();
  const int64_t want = split_wps * num_sms(h);
  int64_t nsplit = std::max<int64_t>(1, (want + ip.wtiles * nbatch - 1) / (ip.wtiles * nbatch));
  nsplit = std::min<int64_t>(nsplit, std::max<int64_t>(1, N / split_min));
  ip.split_len = (N + nsplit - 1) / nsplit;
  ip.nsplit = (N + ip.split_len - 1) / ip.split_len;
  if (ip.nsplit > 1) {
    const int64_t need = nbatch * ip.nsplit * 5 * nt;
    if (need > h->part_cap) {
      drop_graphs(h);
      cudaFree(h->d_part);
      h->d_part = nullptr;
      CU(cudaMalloc(&h->d_part, sizeof(double) * need));
      h->part_cap = need;
    }
  }
  return LANDAU_OK;
}


// Stream-K tables of the per-vertex kernel for a batch of nbatch vertices on S CTAs.  The cuts
// g_c = ceil(c Wtot / S) fall at arbitrary weight offsets; with the canonical round order (pair
// rounds of weight 2, then diagonal rounds of weight 1) a cut inside a pair round gives one CTA a unit
// more than its share (128 C2 vertices: 64 CTAs with 33 of 32 units).  A vertex with cuts inside it
// (split between CTAs anyway) gets its own round order -- rounds of one vertex touch disjoint tiles
// in any order -- built greedily so that every cut offset is a round boundary: from the previous
// boundary s to the cut t, (t - s) mod 2 diagonal rounds and the rest pair rounds.  Vertices without
// inner cuts keep the canonical order (a lone vertex's summation order).  ord [nbatch][R] = round per
// position, wpv [nbatch][R+1] = weight prefix per position.
// per-vertex orders pay where a CTA holds few vertices (the cut imbalance is a unit in ~Wv x vertices
// per CTA); with more, the kernel variant reading the canonical prefix is the faster one (C4 1024
// vertices: 2548 vs 2561 us; 128: 352.8 vs 347.9 us)
bool vtx_use_perv(const landau_t h, int64_t nbatch, int S) {
  static const bool reorder = [] {
    const char *e = getenv("LANDAU_VTX_REORDER");
    return !(e && atoi(e) == 0);
  }();
  return reorder && nbatch < 4LL * S;
}

void vtx_tables(const landau_t h, int64_t nbatch, int S, std::vector<int16_t> &ord, std::vector<int32_t> &wpv) {
  const bool reorder = vtx_use_perv(h, nbatch, S);
  const int R = h->nvtx_rounds;
  const int64_t Wv = h->vtx_Wv, Wtot = nbatch * Wv;
  ord.assign((size_t)nbatch * R, 0);
  wpv.assign((size_t)nbatch * (R + 1), 0);
  std::vector<int> twos, ones;
  for (int r = 0; r < R; r++) (h->vtx_w[r] == 2 ? twos : ones).push_back(r);
  std::vector<int64_t> cuts;
  for (int64_t v = 0; v < nbatch; v++) {
    cuts.clear();   // cut offsets strictly inside vertex v
    const int64_t c0 = (v * Wv * S) / Wtot, c1 = ((v + 1) * Wv * S + Wtot - 1) / Wtot;
    for (int64_t c = std::max<int64_t>(c0, 1); c <= c1; c++) {
      const int64_t g = (c * Wtot + S - 1) / S;
      if (g > v * Wv && g < (v + 1) * Wv) cuts.push_back(g - v * Wv);
    }
    int16_t *o = ord.data() + v * R;
    int n = 0;
    if (cuts.empty() || !reorder) {
      for (int r = 0; r < R; r++) o[n++] = (int16_t)r;
    } else {
      size_t it = 0, io = 0;
      int64_t pos = 0;
      for (int64_t t : cuts) {
        if (t <= pos) continue;
        int64_t need = t - pos;
        int b = (int)(need & 1);
        if (b > (int)(ones.size() - io)) b = 0;
        int64_t a = (need - b) / 2;
        a = std::min<int64_t>(a, (int64_t)(twos.size() - it));
        for (int64_t k = 0; k < a; k++, pos += 2) o[n++] = (int16_t)twos[it++];
        for (int k = 0; k < b; k++, pos += 1) o[n++] = (int16_t)ones[io++];
      }
      while (it < twos.size()) o[n++] = (int16_t)twos[it++];
      while (io < ones.size()) o[n++] = (int16_t)ones[io++];
    }
    int32_t *w = wpv.data() + v * (R + 1);
    w[0] = 0;
    for (int p = 0; p < R; p++) w[p + 1] = w[p] + h->vtx_w[o[p]];
  }
}

int ensure_vtx_tables(landau_t h, int64_t nbatch, int S) {
  if (h->vtx_tab_nb == nbatch && h->vtx_tab_S == S) return LANDAU_OK;
  std::vector<int16_t> ord;
  std::vector<int32_t> wpv;
  vtx_tables(h, nbatch, S, ord, wpv);
  drop_graphs(h);   // captured launches hold the old tables
  cudaFree(h->d_vtx_ord);
  cudaFree(h->d_vtx_wpv);
  h->d_vtx_ord = nullptr;
  h->d_vtx_wpv = nullptr;
  h->vtx_tab_nb = -1;
  int rc;
  if ((rc = upload(h, &h->d_vtx_ord, ord)) || (rc = upload(h, &h->d_vtx_wpv, wpv))) return rc;
  h->vtx_tab_nb = nbatch;
  h->vtx_tab_S = S;
  return LANDAU_OK;
}

int launch_inner(landau_t h, int64_t nbatch) {
  const Plan &P = h->plan;
  const int64_t N = P.npts;
  const int64_t t0 = h->e0 * P.nqp, nt = (h->e1 - h->e0) * P.nqp;
  if (h->tcache) {   // NEXT-4: cached tensors, three FP64 GEMMs
    const int64_t n2 = N * N;
    if (!h->tcache_valid || h->tcache_recompute) {
      dim3 grid((unsigned)((N + 127) / 128), (unsigned)N);
      tensor_fill_kernel<<<grid, 128, 0, h->stream>>>(N, h->d_r, h->d_z, h->d_U, h->d_U + 3 * n2, h->d_U + 5 * n2);
      h->launches++;
      KCHECK();
      h->tcache_valid = true;
    }
    h->stats.nbatch = nbatch;
    h->stats.targets = nt;
    h->stats.sources = N;
    h->stats.inner_path = 2;
    h->stats.nsplit = 1;
    h->stats.pair_evaluations = 0;
    Timer t(h, LANDAU_T_INNER);
    const double one = 1.0, zero = 0.0;
    const int n = (int)N, nb = (int)nbatch;
    double *G = h->d_G;   // [batch][5][N], Nc == N
    int st = g_cublas.Dgemm(h->cublas, 0, 0, 3 * n, nb, n, &one, h->d_U, 3 * n, h->d_wT, 3 * n, &zero, G, 5 * n);
    if (!st) st = g_cublas.Dgemm(h->cublas, 0, 0, n, nb, 2 * n, &one, h->d_U + 3 * n2, n, h->d_wT + N, 3 * n, &zero,
                                 G + 3 * N, 5 * n);
    if (!st) st = g_cublas.Dgemm(h->cublas, 0, 0, n, nb, 2 * n, &one, h->d_U + 5 * n2, n, h->d_wT + N, 3 * n, &zero,
                                 G + 4 * N, 5 * n);
    if (st) return fail(h, LANDAU_ECUDA, "cublasDgemm failed: " + std::to_string(st));
    (void)cudaGetLastError();   // cuBLAS may leave a benign runtime error behind on success
    h->tlaunch[LANDAU_T_INNER] += 1;   // one inner stage (three cuBLAS kernels, not counted as ours)
    return LANDAU_OK;
  }
  InnerPlan ip;
  int rc = inner_plan(h, nbatch, ip);
  if (rc) return rc;
  const int variant = inner_variant();
  const int64_t wtiles = ip.wtiles, nsplit = ip.nsplit, split_len = ip.split_len;
  // [world][batch][5][Nc] chunks (element split), or the one full [batch][5][N] block (pair split)
  double *G_own = h->d_G + (h->dist_pairs ? 0 : (int64_t)h->rank * nbatch * 5 * h->Nc);
  h->stats.nbatch = nbatch;
  h->stats.targets = nt;
  h->stats.sources = N;
  h->stats.inner_path = ip.sym ? 1 : 0;
  h->stats.nsplit = ip.sym ? 1 : ip.nsplit;
  if (ip.sym && h->mirror && h->mirror_on) {
    // tensor evaluations per batch item (this rank's items): U + V items over the T tiles of the upper
    // half; diagonal items 16 (U) + 17 (V) steps x 32 lanes, the others 2 x 32 x 32
    h->stats.pair_evaluations = h->mir_evals;
    h->stats.inner_path = 3;
  } else if (ip.sym) {
    int64_t ev = 0;   // lane-steps per batch item: diagonal items 16 x 32, others 32 x 32 per i-tile
    ev = (int64_t)h->ntiles * 16 * 32 + (int64_t)h->ntiles * (h->ntiles - 1) / 2 * 32 * 32;
    h->stats.pair_evaluations = ev;
  } else {
    h->stats.pair_evaluations = ip.wtiles * 32 * ip.tpt * N;
  }
  // mirror slot kernel over batch items [b0, b0 + nb): partial slots, then their reduction; the item
  // set with runs when the work is ample (>= 16 items per resident warp), single i-tiles otherwise
  auto mir_set = [&](int64_t nb) -> const landau_s::MirSet & {
    const landau_s::MirSet &r = h->mset[1];
    return (r.nitems && nb * r.nitems >= 16LL * kSymWarps * LANDAU_SYM_MINB * num_sms(h)) ? r : h->mset[0];
  };
  auto mir_slots = [&](int64_t b0, int64_t nb) -> int {
    const landau_s::MirSet &ms = mir_set(nb);
    const int64_t nitems = nb * ms.nitems;
    const double *wT = h->d_wT + b0 * 3 * N;
    const unsigned grid = (unsigned)std::min<int64_t>((nitems + kSymWarps - 1) / kSymWarps, (int64_t)LANDAU_SYM_MINB * num_sms(h));
    if (h->coincident)
      inner_mir_kernel<LANDAU_SYM_MINB, true><<<grid, 32 * kSymWarps, 0, h->stream>>>(
          N, h->H, ms.nitems, ms.nslots, nitems, ms.items, h->d_rU, h->d_zU, h->d_pu, h->d_pm, wT, h->d_part);
    else
      inner_mir_kernel<LANDAU_SYM_MINB, false><<<grid, 32 * kSymWarps, 0, h->stream>>>(
          N, h->H, ms.nitems, ms.nslots, nitems, ms.items, h->d_rU, h->d_zU, h->d_pu, h->d_pm, wT, h->d_part);
    h->launches++;
    KCHECK();
    return LANDAU_OK;
  };
  auto mir_reduce = [&](int64_t b0, int64_t nb) -> int {
    const landau_s::MirSet &ms = mir_set(nb);
    Timer t(h, LANDAU_T_REDUCE);
    const int64_t total = nb * 5 * h->H;
    const int blocks = (int)std::min<int64_t>((total + 255) / 256, 16LL * num_sms(h));
    reduce_mir_kernel<<<blocks, 256, 0, h->stream>>>(N, h->H, ms.nslots, ms.tile_ptr, ms.tile_slots, h->d_pu, h->d_pm,
                                                     h->d_part, G_own + b0 * 5 * h->Nc, 5 * h->Nc, (int)nb);
    h->launches++;
    h->tlaunch[LANDAU_T_REDUCE]++;
    KCHECK();
    return LANDAU_OK;
  };
  if (ip.vtx) {   // one CTA per SM, stream-K over the batch's (vertex, round) work, sums in shared memory
    const int64_t T = (h->H + 31) / 32;
    h->stats.pair_evaluations = T * 33 * 32 + 2 * (T * (T - 1) / 2) * 32 * 32;
    h->stats.nsplit = 1;
    h->stats.inner_path = 4;
    VtxSched sc;
    sc.nbatch = (int)nbatch;
    sc.nrounds = h->nvtx_rounds;
    // automatic mode: every SM; mode 3 with a batch below one vertex per SM: one CTA per vertex (no
    // vertex is split: the summation order of a lone build, used by the parity tests)
    sc.S = num_sms(h) * kVtxMinB;
    if (h->mirror_mode == 3 && nbatch < sc.S) sc.S = (int)nbatch;
    sc.Wv = h->vtx_Wv;
    sc.Wtot = nbatch * h->vtx_Wv;
    const bool perv = vtx_use_perv(h, nbatch, sc.S);
    if (perv && (rc = ensure_vtx_tables(h, nbatch, sc.S))) return rc;
    const int32_t *wp = perv ? h->d_vtx_wpv : h->d_vtx_wp;
    const int16_t *ord = perv ? h->d_vtx_ord : nullptr;
    Timer t(h, LANDAU_T_INNER);
#define LAUNCH_VTX(MASK, PERV)                                                                                   \
  inner_vtx_kernel<MASK, PERV><<<sc.S, 32 * kVtxWarps, h->vtx_smem, h->stream>>>(                                \
      N, h->H, sc, h->d_vtx_round_ptr, wp, ord, h->d_vtx_items, h->d_rU, h->d_zU, h->d_pu, h->d_pm, h->d_wT, G_own, \
      5 * h->Nc, h->d_vtx_part, h->d_vtx_cnt)
    if (h->coincident) {
      if (perv) LAUNCH_VTX(true, true);
      else LAUNCH_VTX(true, false);
    } else {
      if (perv) LAUNCH_VTX(false, true);
      else LAUNCH_VTX(false, false);
    }
#undef LAUNCH_VTX
    h->launches++;
    h->tlaunch[LANDAU_T_INNER]++;
    KCHECK();
    return LANDAU_OK;
  }
  if (ip.sym && h->mirror && h->mirror_on) {
    {
      Timer t(h, LANDAU_T_INNER);
      if (mir_set(nbatch).nitems && (rc = mir_slots(0, nbatch))) return rc;
      h->tlaunch[LANDAU_T_INNER]++;
    }
    if ((rc = mir_reduce(0, nbatch))) return rc;
    if (h->dist_pairs) {   // the exchange step: sum the ranks' partial G (every rank gets all of G)
      Timer t(h, LANDAU_T_ALLGATHER);
      h->tlaunch[LANDAU_T_ALLGATHER]++;   // stage count (a NCCL collective, not one of our kernels)
      const int rc2 = g_nccl.AllReduce(G_own, G_own, (size_t)(nbatch * 5 * h->Nc), kNcclFloat64, kNcclSum, h->comm,
                                       h->stream);
      if (rc2 != 0)
        return fail(h, LANDAU_ENCCL, std::string("ncclAllReduce: ") + (g_nccl.GetErrorString ? g_nccl.GetErrorString(rc2) : "error"));
    }
    return LANDAU_OK;
  }
  if (ip.sym) {
    {
      Timer t(h, LANDAU_T_INNER);
      const int64_t nitems = nbatch * h->nsym_items;
      const unsigned grid = (unsigned)std::min<int64_t>((nitems + kSymWarps - 1) / kSymWarps, (int64_t)LANDAU_SYM_MINB * num_sms(h));
      if (h->coincident)   // distinct points share coordinates somewhere: mask every pair (Amb-3)
        inner_sym_kernel<LANDAU_SYM_MINB, true><<<grid, 32 * kSymWarps, 0, h->stream>>>(
            N, h->nsym_items, h->nsym_slots, nitems, h->d_sym_items, h->d_r, h->d_z, h->d_wT, h->d_part);
      else
        inner_sym_kernel<LANDAU_SYM_MINB, false><<<grid, 32 * kSymWarps, 0, h->stream>>>(
            N, h->nsym_items, h->nsym_slots, nitems, h->d_sym_items, h->d_r, h->d_z, h->d_wT, h->d_part);
      h->launches++;
      h->tlaunch[LANDAU_T_INNER]++;
      KCHECK();
    }
    Timer t(h, LANDAU_T_REDUCE);
    const int64_t total = nbatch * 5 * N;
    const int blocks = (int)std::min<int64_t>((total + 255) / 256, 16LL * num_sms(h));
    reduce_sym_kernel<<<blocks, 256, 0, h->stream>>>(N, h->nsym_slots, h->d_tile_ptr, h->d_tile_slots, h->d_part, G_own,
                                                     5 * h->Nc, (int)nbatch);
    h->launches++;
    h->tlaunch[LANDAU_T_REDUCE]++;
    KCHECK();
    return LANDAU_OK;
  }
  if (ip.mdir) {   // mirror-symmetric directed kernel
    const int64_t T = ip.wtiles;
    h->stats.inner_path = 5;
    h->stats.nsplit = nsplit;
    h->stats.pair_evaluations = T * 32 * h->H * 2;   // U + V per (target, source), padded targets
    {
      Timer t(h, LANDAU_T_INNER);
      const int64_t nitems = nbatch * nsplit * T;
      const unsigned grid = (unsigned)((nitems + kMdirWarps - 1) / kMdirWarps);
      inner_mdir_kernel<<<grid, 32 * kMdirWarps, 0, h->stream>>>(N, h->H, T, split_len, (int)nsplit, nitems, h->d_rU,
                                                                 h->d_zU, h->d_pu, h->d_pm, h->d_wT, G_own, 5 * h->Nc,
                                                                 h->d_part);
      h->launches++;
      h->tlaunch[LANDAU_T_INNER]++;
      KCHECK();
    }
    if (nsplit > 1) {
      Timer t(h, LANDAU_T_REDUCE);
      const int blocks = (int)std::min<int64_t>(nbatch * 5 * T, 16LL * num_sms(h));
      reduce_mdir_kernel<<<blocks, 32 * kRedWarps, 0, h->stream>>>(N, h->H, T * 32, (int)nsplit, h->d_pu, h->d_pm, h->d_part, G_own,
                                                        5 * h->Nc, (int)nbatch);
      h->launches++;
      h->tlaunch[LANDAU_T_REDUCE]++;
      KCHECK();
    }
    if (h->comm) {   // LANDAU_DIST_ELEMENTS at world 1: the (trivial) exchange step
      Timer t(h, LANDAU_T_ALLGATHER);
      h->tlaunch[LANDAU_T_ALLGATHER]++;   // stage count (a NCCL collective, not one of our kernels)
      int rc2 = g_nccl.AllGather(G_own, h->d_G, (size_t)(nbatch * 5 * h->Nc), kNcclFloat64, h->comm, h->stream);
      if (rc2 != 0) return fail(h, LANDAU_ENCCL, "ncclAllGather failed");
    }
    return LANDAU_OK;
  }
  double *out;
  int64_t out_bstride;
  if (nsplit == 1) {
    out = G_own;
    out_bstride = 5 * h->Nc;
  } else {
    out = h->d_part;
    out_bstride = nsplit * 5 * nt;
  }
  {
    Timer t(h, LANDAU_T_INNER);
    const int64_t nitems = nbatch * nsplit * wtiles;
    const unsigned grid = (unsigned)((nitems + kInnerWarps - 1) / kInnerWarps);
#define LAUNCH_INNER(T, M)                                                                              \
  inner_kernel<T, M><<<grid, kInnerTB, 0, h->stream>>>(N, t0, nt, split_len, (int)nsplit, wtiles, nitems, h->d_r, h->d_z, \
                                                      h->d_wT, out, out_bstride)
    switch (variant) {
      case 0: LAUNCH_INNER(1, 3); break;
      case 1: LAUNCH_INNER(2, 2); break;
      case 4: LAUNCH_INNER(4, 2); break;
      default: LAUNCH_INNER(2, 3); break;
    }
#undef LAUNCH_INNER
    h->launches++;
    h->tlaunch[LANDAU_T_INNER]++;
    KCHECK();
  }
  if (nsplit > 1) {
    Timer t(h, LANDAU_T_REDUCE);
    const int64_t total = nbatch * 5 * nt;
    const int blocks = (int)std::min<int64_t>((total + 255) / 256, 16LL * num_sms(h));
    // G_own is [batch][5][Nc] with Nc >= nt
    reduce_kernel<<<blocks, 256, 0, h->stream>>>(nt, (int)nsplit, h->d_part, G_own, 5 * h->Nc, (int)nbatch);
    h->launches++;
    h->tlaunch[LANDAU_T_REDUCE]++;
    KCHECK();
  }
  if (h->comm) {   // LANDAU_DIST_ELEMENTS: the exchange step (also run at world == 1)
    Timer t(h, LANDAU_T_ALLGATHER);
      h->tlaunch[LANDAU_T_ALLGATHER]++;   // stage count (a NCCL collective, not one of our kernels)
    int rc = g_nccl.AllGather(G_own, h->d_G, (size_t)(nbatch * 5 * h->Nc), kNcclFloat64, h->comm, h->stream);
    if (rc != 0) return fail(h, LANDAU_ENCCL, std::string("ncclAllGather: ") + (g_nccl.GetErrorString ? g_nccl.GetErrorString(rc) : "error"));
  }
  return LANDAU_OK;
}

template <int NB>
int launch_element(landau_t h, int64_t nbatch, int64_t b0, int64_t nb) {
  const Plan &P = h->plan;
  Timer t(h, LANDAU_T_ELEMENT);
  constexpr int S = NB == 9 ? 3 : (NB == 16 ? 4 : 5);
#ifndef LANDAU_EL_EPB16
#define LANDAU_EL_EPB16 8
#endif
  constexpr int EPB = NB == 9 ? 14 : (NB == 16 ? LANDAU_EL_EPB16 : 5);   // ~128 threads per block
  static const bool sf = [] {
    const char *e = getenv("LANDAU_ELEMENT_SF");
    return !(e && atoi(e) == 0);
  }();
  if (sf && P.ncell * nb < (1LL << 32)) {   // sum factorisation, one warp per cell
    const int64_t items = P.ncell * nb;
    static const int64_t sf_bps = [] {   // grid cap in blocks per SM (LANDAU_SF_BLOCKS_PER_SM)
      const char *e = getenv("LANDAU_SF_BLOCKS_PER_SM");
      return e ? (int64_t)atoll(e) : (int64_t)64;   // C4: 64 0.113 ms, 16 0.118 ms
    }();
    const unsigned grid = (unsigned)std::min<int64_t>((items + kSfWarps - 1) / kSfWarps, sf_bps * num_sms(h));
    element_sf_kernel<S><<<grid, 32 * kSfWarps, 0, h->stream>>>(P.ncell, h->d_G, h->Nc, (int)nbatch, (int)b0, (int)nb,
                                                               h->d_w, h->d_h, h->d_tab + 3 * NB * NB, h->d_C);
  } else {
    const int64_t items = (P.ncell + EPB - 1) / EPB * nb;
    const unsigned grid = (unsigned)std::min<int64_t>(items, 16LL * num_sms(h));
    element_kernel<NB, S, EPB><<<grid, NB * EPB, 0, h->stream>>>(P.ncell, h->d_G, h->Nc, (int)nbatch, (int)b0, (int)nb,
                                                                  h->d_w, h->d_h, h->d_tab, h->d_C);
  }
  h->launches++;
  h->tlaunch[LANDAU_T_ELEMENT]++;
  KCHECK();
  return LANDAU_OK;
}

template <int NB>
int launch_assemble(landau_t h, int64_t nbatch, double *out, int format) {   // nbatch = items in the chunk
  const Plan &P = h->plan;
  Timer t(h, LANDAU_T_ASSEMBLE);
  const int64_t out_bstride = format == LANDAU_CSR ? h->nnz : h->ncoo;
  for (int g = 0; g < P.ngrids; g++) {
    const auto &m = format == LANDAU_CSR ? h->d_csr[g] : h->d_coo[g];
    GatherDev gd;
    gd.ptr = m.ptr;
    gd.idx = m.idx;
    gd.w = m.w;
    gd.nslots = m.nslots;
    gd.nsp = h->spc.grid_nsp[g];
    for (int q = 0; q < h->spc.grid_nsp[g]; q++) {
      int sp = h->spc.grid_sp[g][q];
      gd.out_off[q] = format == LANDAU_CSR ? h->snnz_off[sp] : h->scoo_off[sp];
      gd.fD[q] = h->spc.fD[sp];
      gd.fK[q] = h->spc.fK[sp];
    }
    if (h->spc.grid_nsp[g] == 0 || m.nslots == 0) continue;
    static const int bpt = [] {   // batch items per thread (LANDAU_ASM_BPT 1/2/4/8/16; C4: 4 0.191 ms, 8 0.201, 2 0.208, 16 0.453)
      const char *e = getenv("LANDAU_ASM_BPT");
      return e ? atoi(e) : 4;
    }();
#define LAUNCH_ASM(BPT)                                                                                          \
  assemble_kernel<NB, BPT><<<dim3((unsigned)((m.nslots + 127) / 128), (unsigned)((nbatch + BPT - 1) / BPT)), 128, 0, \
                             h->stream>>>(gd, h->d_C, P.ncell * 2 * NB * NB, out, out_bstride, (int)nbatch)
    if (bpt == 4) LAUNCH_ASM(4);
    else if (bpt == 2) LAUNCH_ASM(2);
    else if (bpt == 1) LAUNCH_ASM(1);
    else if (bpt == 16) LAUNCH_ASM(16);
    else LAUNCH_ASM(8);
#undef LAUNCH_ASM
    h->launches++;
    h->tlaunch[LANDAU_T_ASSEMBLE]++;
    KCHECK();
  }
  return LANDAU_OK;
}

template <int NB>
int launch_tail(landau_t h, int64_t nbatch, double *out, int format) {
  const Plan &P = h->plan;
  constexpr int S = NB == 9 ? 3 : (NB == 16 ? 4 : 5);
  Timer t(h, LANDAU_T_ELEMENT);   // a-4 and a-5 in one kernel: timed as the element stage
  const int64_t out_bstride = format == LANDAU_CSR ? h->nnz : h->ncoo;
  const auto &m = h->tmaps[format == LANDAU_CSR ? 0 : 1];
  TailDev td{m.grid_phase_ptr,
             m.cell_ptr,
             m.slot_ptr,
             reinterpret_cast<const int2 *>(m.meta),
             reinterpret_cast<const int2 *>(m.optr),
             reinterpret_cast<const int4 *>(m.idx4),
             reinterpret_cast<const double2 *>(m.w4),
             m.oidx,
             m.ow,
             P.ngrids,
             m.nphases,
             m.max_cells,
             m.max_cross};
  const size_t smem = tail_smem_bytes<S>(m.max_cells, m.max_cross);
  // > 48 KB of dynamic shared memory: the attribute is per device and cheap to set, so on every call
  CU(cudaFuncSetAttribute(tail_kernel<S>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  tail_kernel<S><<<(unsigned)tail_grid(h, nbatch), 32 * tail_warps<S>(), smem, h->stream>>>(
      h->d_G, P.npts, (int)nbatch, h->d_w, h->d_h, h->d_tab + 3 * NB * NB, td, h->d_gmaps[format == LANDAU_CSR ? 0 : 1],
      out, out_bstride);
  h->launches++;
  h->tlaunch[LANDAU_T_ELEMENT]++;
  KCHECK();
  return LANDAU_OK;
}

// Whole small builds as ONE cooperative launch (kernels_single.cuh): the mirror-directed path of single
// builds / tiny batches on Q2-Q3 meshes, CSR or COO, when no per-stage timers are requested.
// LANDAU_FUSED_SINGLE=0 disables it.
bool fused_single_enabled() {
  static const bool v = [] {
    const char *e = getenv("LANDAU_FUSED_SINGLE");
    return !(e && atoi(e) == 0);
  }();
  return v;
}

bool fused_single_ok(landau_t h, int64_t nbatch) {
  // latency-bound builds only: at most one target tile per SM (C2: up to 8 vertices)
  return fused_single_enabled() && h->plan.nb <= 16 && !h->timing && !h->comm && !h->tcache && h->world == 1 &&
         h->Nc == h->plan.npts && nbatch <= h->chunk && h->mirror && h->mirror_on &&
         nbatch * ((h->H + 31) / 32) <= num_sms(h);
}

template <int NB>
int launch_single(landau_t h, int64_t nbatch, const InnerPlan &ip, double *out, int format) {
  if constexpr (NB > 16) {
    return fail(h, LANDAU_EUNSUPPORTED, "fused single build: Q2/Q3 only");
  } else {
    const Plan &P = h->plan;
    SingleBuildArgs a{};
    a.ncell = P.ncell;
    a.ndof_total = h->ndof;
    a.nbatch = (int)nbatch;
    a.f = h->fin ? h->fin : h->d_f;
    a.ext_ptr = h->d_ext_ptr;
    a.ext_dof = h->d_ext_dof;
    a.ext_w = h->d_ext_w;
    a.cell_grid = h->d_cell_grid;
    a.cell_h = h->d_h;
    a.pw = h->d_w;
    a.tab = h->d_tab;
    a.tab1 = h->d_tab + 3 * NB * NB;
    a.sp = h->spc;
    a.wT = h->d_wT;
    a.npts = P.npts;
    a.H = h->H;
    a.T = ip.wtiles;
    a.split_len = ip.split_len;
    a.nsplit = (int)ip.nsplit;
    a.rU = h->d_rU;
    a.zU = h->d_zU;
    a.pu = h->d_pu;
    a.pm = h->d_pm;
    a.pinv = h->d_pinv;
    a.G = h->d_G;
    a.part = h->d_part;
    a.Cbuf = h->d_C;
    a.maps = h->d_gmaps[format == LANDAU_CSR ? 0 : 1];
    a.ngrids = P.ngrids;
    a.out = out;
    a.out_bstride = format == LANDAU_CSR ? h->nnz : h->ncoo;
    const int64_t inner_items = nbatch * ip.wtiles * ((ip.nsplit + kSbWarps - 1) / kSbWarps);   // CTA items
    const unsigned grid = (unsigned)std::max<int64_t>(1, std::min<int64_t>(num_sms(h), inner_items));
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(grid);
    cfg.blockDim = dim3(32 * kSbWarps);
    cfg.dynamicSmemBytes = 0;
    cfg.stream = h->stream;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeCooperative;
    attr[0].val.cooperative = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    CU(cudaLaunchKernelEx(&cfg, single_build_kernel<NB>, a));
    h->launches++;
    h->stats.nbatch = nbatch;
    h->stats.targets = P.npts;
    h->stats.sources = P.npts;
    h->stats.inner_path = 5;
    h->stats.nsplit = ip.nsplit;
    h->stats.pair_evaluations = ip.wtiles * 32 * h->H * 2;
    return LANDAU_OK;
  }
}

template <int NB>
int build_jacobian(landau_t h, int64_t nbatch, double *out, int format) {
  int rc;
  if (out && fused_single_ok(h, nbatch)) {
    InnerPlan ip;
    if ((rc = inner_plan(h, nbatch, ip))) return rc;
    if (ip.mdir && !ip.vtx && !ip.sym) return launch_single<NB>(h, nbatch, ip, out, format);
  }
  if ((rc = launch_field<NB>(h, nbatch))) return rc;
  if ((rc = launch_inner(h, nbatch))) return rc;
  if (!out) return LANDAU_OK;   // point_coeffs: G only
  if (use_tail(h, nbatch)) return launch_tail<NB>(h, nbatch, out, format);
  // a-4 + a-5 in batch chunks whose element matrices stay resident in L2 between the two kernels
  const int64_t nb = h->chunk;
  const int64_t out_bstride = format == LANDAU_CSR ? h->nnz : h->ncoo;
  for (int64_t b0 = 0; b0 < nbatch; b0 += nb) {
    const int64_t n = std::min(nb, nbatch - b0);
    if ((rc = launch_element<NB>(h, nbatch, b0, n))) return rc;
    if ((rc = launch_assemble<NB>(h, n, out + b0 * out_bstride, format))) return rc;
  }
  return LANDAU_OK;
}

int dispatch_build_direct(landau_t h, int64_t nbatch, double *out, int format) {
  switch (h->plan.nb) {
    case 9: return build_jacobian<9>(h, nbatch, out, format);
    case 16: return build_jacobian<16>(h, nbatch, out, format);
    case 25: return build_jacobian<25>(h, nbatch, out, format);
  }
  return fail(h, LANDAU_EUNSUPPORTED, "order");
}

// A whole build replays as one CUDA graph (launch-latency bound for small meshes) unless per-stage
// timers are on, the legacy default stream is in use, or the build has a collective.
int dispatch_build(landau_t h, int64_t nbatch, double *out, int format) {
  if (h->timing || !h->use_graphs || !h->stream || h->comm || !out || h->tcache)
    return dispatch_build_direct(h, nbatch, out, format);
  for (auto &g : h->graphs)
    if (g.nbatch == nbatch && g.format == format && g.out == out && g.fin == h->fin) {
      CU(cudaGraphLaunch(g.exec, h->stream));
      h->launches += g.kernels;
      return LANDAU_OK;
    }
  InnerPlan ip;   // allocate everything before capturing
  int rc = inner_plan(h, nbatch, ip);
  if (rc) return rc;
  const int64_t l0 = h->launches;
  int64_t tl[LANDAU_NTIMERS];
  memcpy(tl, h->tlaunch, sizeof tl);
  CU(cudaStreamBeginCapture(h->stream, cudaStreamCaptureModeThreadLocal));
  rc = dispatch_build_direct(h, nbatch, out, format);
  cudaGraph_t graph = nullptr;
  cudaError_t ce = cudaStreamEndCapture(h->stream, &graph);
  const int64_t kernels = h->launches - l0;
  h->launches = l0;
  memcpy(h->tlaunch, tl, sizeof tl);
  if (rc) {
    if (graph) cudaGraphDestroy(graph);
    return rc;
  }
  if (ce != cudaSuccess) return fail(h, LANDAU_ECUDA, std::string("graph capture: ") + cudaGetErrorString(ce));
  cudaGraphExec_t exec = nullptr;
  ce = cudaGraphInstantiate(&exec, graph, 0);
  cudaGraphDestroy(graph);
  if (ce != cudaSuccess) return fail(h, LANDAU_ECUDA, std::string("graph instantiate: ") + cudaGetErrorString(ce));
  if (h->graphs.size() >= 32) {   // (landau_jacobian_host keeps one graph per chunk: up to 16)
    cudaGraphExecDestroy(h->graphs.front().exec);
    h->graphs.erase(h->graphs.begin());
  }
  h->graphs.push_back({nbatch, format, out, h->fin, exec, kernels});
  CU(cudaGraphLaunch(exec, h->stream));
  h->launches += kernels;
  return LANDAU_OK;
}

template <int NB>
int build_mass(landau_t h) {
  const Plan &P = h->plan;
  double *Mbuf = nullptr;
  CU(cudaMalloc(&Mbuf, sizeof(double) * P.ncell * 2 * NB * NB));
  mass_element_kernel<NB><<<(unsigned)P.ncell, NB * NB, 0, h->stream>>>(P.ncell, h->d_w, h->d_h, h->d_tab, Mbuf);
  h->launches++;
  KCHECK();
  for (int g = 0; g < P.ngrids; g++) {
    for (int f = 0; f < 4; f++) {   // mass CSR, mass COO, advection CSR, advection COO
      const auto &m = f % 2 == 0 ? h->d_csr[g] : h->d_coo[g];
      double *&dst = f == 0 ? h->d_mass_csr[g] : f == 1 ? h->d_mass_coo[g] : f == 2 ? h->d_adv_csr[g] : h->d_adv_coo[g];
      CU(cudaMalloc(&dst, sizeof(double) * std::max<int64_t>(m.nslots, 1)));
      if (m.nslots == 0) continue;
      mass_gather_kernel<<<(unsigned)((m.nslots + 255) / 256), 256, 0, h->stream>>>(m.ptr, m.idx, m.w, m.nslots,
                                                                                    Mbuf + (f < 2 ? 0 : 1), dst);
      h->launches++;
      KCHECK();
    }
  }
  CU(cudaStreamSynchronize(h->stream));
  cudaFree(Mbuf);
  return LANDAU_OK;
}

// The dynamic shared-memory limit of inner_vtx_kernel is a per-function attribute shared by every
// handle on a device, so it only ever grows: the largest need of any handle created so far (setting a
// small handle's size would make a larger handle's launches fail).
bool raise_vtx_smem_attr(int device, size_t bytes) {
  static std::mutex mu;
  static size_t cur[64] = {0};
  std::lock_guard<std::mutex> lk(mu);
  size_t &c = cur[device & 63];
  if (bytes <= c) return true;
  if (cudaFuncSetAttribute(inner_vtx_kernel<true, false>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)bytes) != cudaSuccess ||
      cudaFuncSetAttribute(inner_vtx_kernel<false, false>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)bytes) != cudaSuccess ||
      cudaFuncSetAttribute(inner_vtx_kernel<true, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)bytes) != cudaSuccess ||
      cudaFuncSetAttribute(inner_vtx_kernel<false, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)bytes) != cudaSuccess)
    return false;
  c = bytes;
  return true;
}

// Mirror symmetry z -> -z: every grid's quadrature points pair up as (r, z), (r, -z)
// BIT-EXACTLY (no point on z = 0).  The mirror kernels evaluate the tensors of a point's mirror from
// the point itself, so anything short of bit-exact equality would move the caller's points; meshes
// that are symmetric only up to rounding take the general kernels.  pu: upper-half points (z > 0),
// pm: their mirrors, grid by grid, each grid's pairs sorted by (r, z).
bool detect_mirror(const Plan &P, std::vector<int32_t> &pu, std::vector<int32_t> &pm) {
  pu.clear();
  pm.clear();
  for (int g = 0; g < P.ngrids; g++) {
    const GridPlan &G = P.grids[g];
    std::vector<int64_t> up, lo;
    for (int64_t i = G.pt0; i < G.pt0 + G.ncell * P.nqp; i++) {
      if (P.pz[i] > 0) up.push_back(i);
      else if (P.pz[i] < 0) lo.push_back(i);
      else return false;   // a point on z = 0 would be its own mirror
    }
    if (up.size() != lo.size()) return false;
    auto by_rz = [&](int64_t a, int64_t b) { return P.pr[a] != P.pr[b] ? P.pr[a] < P.pr[b] : P.pz[a] < P.pz[b]; };
    auto by_rmz = [&](int64_t a, int64_t b) { return P.pr[a] != P.pr[b] ? P.pr[a] < P.pr[b] : -P.pz[a] < -P.pz[b]; };
    std::sort(up.begin(), up.end(), by_rz);
    std::sort(lo.begin(), lo.end(), by_rmz);
    for (size_t k = 0; k < up.size(); k++) {
      const int64_t a = up[k], b = lo[k];
      if (P.pr[a] != P.pr[b] || P.pz[b] != -P.pz[a]) return false;
      if (k && P.pr[a] == P.pr[up[k - 1]] && P.pz[a] == P.pz[up[k - 1]]) return false;   // twins
      pu.push_back((int32_t)a);
      pm.push_back((int32_t)b);
    }
  }
  return !pu.empty();
}

// Every C entry point runs its body through guarded(): the header promises that nothing throws or
// aborts, so a std::bad_alloc (host vectors of a large mesh or batch) becomes LANDAU_ENOMEM and any
// other exception LANDAU_EINVAL, and a handle's calls run on the handle's device whatever device is
// current in the calling thread (restored afterwards).
struct DeviceGuard {
  int prev = -1;
  explicit DeviceGuard(landau_t h) {
    int cur = 0;
    if (h && !h->host_only && cudaGetDevice(&cur) == cudaSuccess && cur != h->device && cudaSetDevice(h->device) == cudaSuccess)
      prev = cur;
  }
  ~DeviceGuard() {
    if (prev >= 0) cudaSetDevice(prev);
  }
};

template <class F>
int guarded(landau_t h, F &&body) {
  try {
    DeviceGuard g(h);
    return body();
  } catch (const std::bad_alloc &) {
    return fail(h, LANDAU_ENOMEM, "host allocation failed (std::bad_alloc)");
  } catch (const std::exception &e) {
    return fail(h, LANDAU_EINVAL, std::string("exception: ") + e.what());
  } catch (...) {
    return fail(h, LANDAU_EINVAL, "unknown exception");
  }
}

}  // namespace

// ==================================================================================================
// C ABI
// ==================================================================================================
static int create_impl(landau_t &h, landau_t *out, const landau_mesh_t *mesh, const landau_params_t *prm,
                       int32_t cuda_device, void *cuda_stream, const landau_dist_t *dist);

extern "C" {

const char *landau_version(void) { return "landau-b200 0.1 (sm_100a, FP64)"; }

const char *landau_strerror(int code) {
  switch (code) {
    case LANDAU_OK: return "ok";
    case LANDAU_EINVAL: return "invalid argument";
    case LANDAU_ENOMEM: return "out of memory";
    case LANDAU_ECUDA: return "CUDA error";
    case LANDAU_ENCCL: return "NCCL error";
    case LANDAU_ESTATE: return "no state set (or batch size mismatch)";
    case LANDAU_EUNSUPPORTED: return "unsupported";
  }
  return "unknown error";
}

const char *landau_last_error(landau_t h) { return h ? h->err.c_str() : g_create_error.c_str(); }

int landau_partition(int64_t nelem, int32_t world, int32_t rank, int64_t *e0, int64_t *e1) {
  return guarded(nullptr, [&]() -> int {
  if (nelem < 0 || world < 1 || rank < 0 || rank >= world || !e0 || !e1) return LANDAU_EINVAL;
  const int64_t chunk = (nelem + world - 1) / world;
  *e0 = std::min<int64_t>(nelem, (int64_t)rank * chunk);
  *e1 = std::min<int64_t>(nelem, (int64_t)(rank + 1) * chunk);
  return LANDAU_OK;
});
}

int landau3d_inner(int64_t n, const double *xyz_dev, const double *wTD_dev, const double *wTK_dev, double *G_dev,
                   void *cuda_stream) {
  return guarded(nullptr, [&]() -> int {
  if (n < 0 || (n > 0 && (!xyz_dev || !wTD_dev || !wTK_dev || !G_dev))) return LANDAU_EINVAL;
  if (n == 0) return LANDAU_OK;
  cudaStream_t st = (cudaStream_t)cuda_stream;
  int dev = 0, sms = 148;
  if (cudaGetDevice(&dev) != cudaSuccess || cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev) != cudaSuccess)
    return LANDAU_ECUDA;
  static const int tpt = [] {   // targets per lane (LANDAU_3D_TPT: 1, 2 or 4)
    const char *e = getenv("LANDAU_3D_TPT");
    return e ? atoi(e) : 2;
  }();
  const int TPT = tpt == 1 || tpt == 4 ? tpt : 2;
  const int64_t wtiles = (n + 32 * TPT - 1) / (32 * TPT);
  int64_t nsplit = std::max<int64_t>(1, (12LL * sms + wtiles - 1) / wtiles);   // >= 12 warps per SM
  nsplit = std::min<int64_t>(nsplit, std::max<int64_t>(1, n / 32));
  const int64_t split_len = (n + nsplit - 1) / nsplit;
  nsplit = (n + split_len - 1) / split_len;
  double *part = G_dev;
  if (nsplit > 1 && cudaMallocAsync((void **)&part, sizeof(double) * nsplit * 9 * n, st) != cudaSuccess) return LANDAU_ENOMEM;
  const int64_t nitems = nsplit * wtiles;
  const unsigned grid3 = (unsigned)((nitems + k3dWarps - 1) / k3dWarps);
  if (TPT == 1)
    inner3d_kernel<1><<<grid3, 32 * k3dWarps, 0, st>>>(n, split_len, (int)nsplit, wtiles, nitems, xyz_dev, wTD_dev, wTK_dev, part);
  else if (TPT == 4)
    inner3d_kernel<4><<<grid3, 32 * k3dWarps, 0, st>>>(n, split_len, (int)nsplit, wtiles, nitems, xyz_dev, wTD_dev, wTK_dev, part);
  else
    inner3d_kernel<2><<<grid3, 32 * k3dWarps, 0, st>>>(n, split_len, (int)nsplit, wtiles, nitems, xyz_dev, wTD_dev, wTK_dev, part);
  cudaError_t e = cudaGetLastError();
  if (nsplit > 1) {
    if (e == cudaSuccess) {
      reduce3d_kernel<<<(unsigned)std::min<int64_t>((9 * n + 255) / 256, 16LL * sms), 256, 0, st>>>(n, (int)nsplit, part, G_dev);
      e = cudaGetLastError();
    }
    cudaFreeAsync(part, st);
  }
  return e == cudaSuccess ? LANDAU_OK : LANDAU_ECUDA;
});
}

int landau_pair_partition(int64_t ntiles, int32_t world, int32_t rank, int64_t *q0, int64_t *q1) {
  return guarded(nullptr, [&]() -> int {
  if (ntiles < 0 || world < 1 || rank < 0 || rank >= world || !q0 || !q1) return LANDAU_EINVAL;
  // items in the slot kernel's order (b = 0.., a = 0..b), weight 2 per pair, 1 per diagonal item
  // (half the steps); rank r takes the items whose weight prefix lies in [r W / world, (r+1) W / world)
  const int64_t nitems = ntiles * (ntiles + 1) / 2, wtot = ntiles * ntiles;   // 2 T(T-1)/2 + T
  const int64_t w0 = wtot * rank / world, w1 = wtot * (rank + 1) / world;
  int64_t q = 0, acc = 0, lo = -1, hi = nitems;
  for (int64_t b = 0; b < ntiles; b++)
    for (int64_t a = 0; a <= b; a++, q++) {
      if (lo < 0 && acc >= w0) lo = q;
      if (acc >= w1) {
        hi = q;
        b = ntiles;
        break;
      }
      acc += a == b ? 1 : 2;
    }
  *q0 = lo < 0 ? nitems : lo;
  *q1 = std::max(*q0, hi);
  return LANDAU_OK;
});
}

int landau_nccl_unique_id(void *out128) {
  return guarded(nullptr, [&]() -> int {
  if (!out128) return LANDAU_EINVAL;
  if (!load_nccl()) return LANDAU_ENCCL;
  ncclUniqueId_ id;
  if (g_nccl.GetUniqueId(&id) != 0) return LANDAU_ENCCL;
  memcpy(out128, &id, 128);
  return LANDAU_OK;
});
}

int landau_create(landau_t *out, const landau_mesh_t *mesh, const landau_params_t *prm, int32_t cuda_device,
                  void *cuda_stream, const landau_dist_t *dist) {
  landau_t h = nullptr;
  int rc, prev_dev = -1;
  if (cuda_device != LANDAU_HOST_ONLY && cudaGetDevice(&prev_dev) != cudaSuccess) prev_dev = -1;
  try {
    rc = create_impl(h, out, mesh, prm, cuda_device, cuda_stream, dist);
  } catch (const std::bad_alloc &) {
    rc = fail(nullptr, LANDAU_ENOMEM, "landau_create: host allocation failed (std::bad_alloc)");
  } catch (const std::exception &e) {
    rc = fail(nullptr, LANDAU_EINVAL, std::string("landau_create: ") + e.what());
  } catch (...) {
    rc = fail(nullptr, LANDAU_EINVAL, "landau_create: unknown exception");
  }
  if (rc && h) {   // a throw left a partly built handle behind
    const std::string m = g_create_error;
    landau_destroy(h);
    g_create_error = m;
    if (out) *out = nullptr;
  }
  if (prev_dev >= 0) cudaSetDevice(prev_dev);   // the caller's current device is left as it was
  return rc;
}

void landau_destroy(landau_t h) {
  try {
  if (!h) return;
  if (h->host_only) {
    delete h;
    return;
  }
  cudaSetDevice(h->device);
  if (h->stream) cudaStreamSynchronize(h->stream);
  drop_graphs(h);
  if (h->cublas && g_cublas.Destroy) g_cublas.Destroy(h->cublas);
  cudaFree(h->d_U);
  for (int32_t *p : h->d_ent_ptr) cudaFree(p);
  for (int32_t *p : h->d_ent_slot) cudaFree(p);
  for (uint16_t *p : h->d_ent_pos) cudaFree(p);
  cudaFree(h->d_Aent);
  cudaFree(h->d_band_desc);
  cudaFree(h->d_perm_all);
  cudaFree(h->d_perm_off);
  cudaFree(h->d_vec_off);
  cudaFree(h->d_band);
  cudaFree(h->d_yfwd);
  if (h->s_h2d) cudaStreamDestroy(h->s_h2d);
  if (h->s_d2h) cudaStreamDestroy(h->s_d2h);
  for (auto e : h->ev_h2d) cudaEventDestroy(e);
  for (auto e : h->ev_built) cudaEventDestroy(e);
  if (h->comm && g_nccl.CommDestroy) g_nccl.CommDestroy(h->comm);
  for (double *p : {h->d_r, h->d_z, h->d_w, h->d_h, h->d_tab, h->d_ext_w, h->d_f, h->d_wT, h->d_part, h->d_G, h->d_C, h->d_vals_tmp})
    cudaFree(p);
  cudaFree(h->d_cell_grid);
  cudaFree(h->d_sym_items);
  cudaFree(h->d_tile_ptr);
  cudaFree(h->d_tile_slots);
  cudaFree(h->d_rU);
  cudaFree(h->d_zU);
  cudaFree(h->d_pu);
  cudaFree(h->d_pinv);
  cudaFree(h->d_pm);
  for (auto &ms : h->mset) {
    cudaFree(ms.items);
    cudaFree(ms.tile_ptr);
    cudaFree(ms.tile_slots);
  }
  cudaFree(h->d_vtx_items);
  cudaFree(h->d_vtx_round_ptr);
  cudaFree(h->d_gmaps[0]);
  cudaFree(h->d_gmaps[1]);
  for (auto &m : h->tmaps)
    for (void *q : {(void *)m.grid_phase_ptr, (void *)m.cell_ptr, (void *)m.slot_ptr, (void *)m.meta, (void *)m.idx4,
                    (void *)m.optr, (void *)m.oidx, (void *)m.w4, (void *)m.ow})
      cudaFree(q);
  cudaFree(h->d_vtx_wp);
  cudaFree(h->d_vtx_ord);
  cudaFree(h->d_vtx_wpv);
  cudaFree(h->d_vtx_part);
  cudaFree(h->d_vtx_cnt);
  cudaFree(h->d_ext_ptr);
  cudaFree(h->d_ext_dof);
  for (auto *v : {&h->d_csr, &h->d_coo})
    for (auto &m : *v) {
      cudaFree(m.ptr);
      cudaFree(m.idx);
      cudaFree(m.w);
    }
  for (double *p : h->d_mass_csr) cudaFree(p);
  for (double *p : h->d_mass_coo) cudaFree(p);
  for (double *p : h->d_adv_csr) cudaFree(p);
  for (double *p : h->d_adv_coo) cudaFree(p);
  for (int64_t *p : h->d_rowptr) cudaFree(p);
  for (int32_t *p : h->d_col) cudaFree(p);
  cudaFree(h->d_Jwork);
  cudaFree(h->d_rhs);
  cudaFree(h->d_norms);
  cudaFree(h->d_srcx);
  if (h->h_norms) cudaFreeHost(h->h_norms);
  for (auto &u : h->ev_used) {
    cudaEventDestroy(u.second.first);
    cudaEventDestroy(u.second.second);
  }
  for (auto e : h->ev_pool) cudaEventDestroy(e);
  (void)cudaGetLastError();   // teardown leaves no error behind for the next call
  delete h;
  } catch (...) {   // teardown never throws out of the C ABI
  }
}

int landau_get_sizes(landau_t h, int64_t *ndof, int64_t *npoints, int64_t *nnz_csr, int64_t *ncoo) {
  return guarded(h, [&]() -> int {
  if (!h) return LANDAU_EINVAL;
  if (ndof) *ndof = h->ndof;
  if (npoints) *npoints = h->plan.npts;
  if (nnz_csr) *nnz_csr = h->nnz;
  if (ncoo) *ncoo = h->ncoo;
  return LANDAU_OK;
});
}

int landau_get_grid_ndof(landau_t h, int32_t grid, int64_t *ndof) {
  return guarded(h, [&]() -> int {
  if (!h || !ndof || grid < 0 || grid >= h->plan.ngrids) return LANDAU_EINVAL;
  *ndof = h->plan.grids[grid].ndof;
  return LANDAU_OK;
});
}

int landau_get_nodes(landau_t h, int32_t grid, double *r, double *z) {
  return guarded(h, [&]() -> int {
  if (!h || grid < 0 || grid >= h->plan.ngrids) return LANDAU_EINVAL;
  const auto &G = h->plan.grids[grid];
  if (r) memcpy(r, G.node_r.data(), sizeof(double) * G.ndof);
  if (z) memcpy(z, G.node_z.data(), sizeof(double) * G.ndof);
  return LANDAU_OK;
});
}

int landau_get_points(landau_t h, double *r, double *z, double *w) {
  return guarded(h, [&]() -> int {
  if (!h) return LANDAU_EINVAL;
  const Plan &P = h->plan;
  if (r) memcpy(r, P.pr.data(), sizeof(double) * P.npts);
  if (z) memcpy(z, P.pz.data(), sizeof(double) * P.npts);
  if (w) memcpy(w, P.pw.data(), sizeof(double) * P.npts);
  return LANDAU_OK;
});
}

int landau_get_pattern(landau_t h, int64_t *csr_rowptr, int32_t *csr_col, int32_t *coo_row, int32_t *coo_col) {
  return guarded(h, [&]() -> int {
  if (!h) return LANDAU_EINVAL;
  const Plan &P = h->plan;
  int64_t row = 0, k = 0, kc = 0;
  if (csr_rowptr) csr_rowptr[0] = 0;
  for (int a = 0; a < h->S; a++) {
    const GridPlan &G = P.grids[h->sgrid[a]];
    const int64_t off = h->soff[a];
    for (int i = 0; i < G.ndof; i++, row++) {
      for (int64_t q = G.rowptr[i]; q < G.rowptr[i + 1]; q++, k++)
        if (csr_col) csr_col[k] = (int32_t)(off + G.col[q]);
      if (csr_rowptr) csr_rowptr[row + 1] = k;
    }
    for (int64_t c = 0; c < G.ncell; c++) {
      const int ne = G.ne[c];
      const int *d = &G.edof[G.edof_off[c]];
      for (int i = 0; i < ne; i++)
        for (int j = 0; j < ne; j++, kc++) {
          if (coo_row) coo_row[kc] = (int32_t)(off + d[i]);
          if (coo_col) coo_col[kc] = (int32_t)(off + d[j]);
        }
    }
  }
  return LANDAU_OK;
});
}

int landau_set_state_batched(landau_t h, int64_t nbatch, const double *f_dev) {
  return guarded(h, [&]() -> int {
  if (h && h->host_only) return fail(h, LANDAU_EUNSUPPORTED, "host-only handle");
  if (!h || nbatch < 1 || !f_dev) return fail(h, LANDAU_EINVAL, "set_state: bad argument");
  int rc = ensure_workspace(h, nbatch);
  if (rc) return rc;
  CU(cudaMemcpyAsync(h->d_f, f_dev, sizeof(double) * nbatch * h->ndof, cudaMemcpyDeviceToDevice, h->stream));
  h->nbatch = nbatch;
  h->have_state = true;
  return LANDAU_OK;
});
}

int landau_set_state(landau_t h, const double *f_dev) {
  return guarded(h, [&]() -> int { return landau_set_state_batched(h, 1, f_dev); });
}

int landau_jacobian_batched(landau_t h, int64_t nbatch, double *values_dev, int32_t format) {
  return guarded(h, [&]() -> int {
  if (h && h->host_only) return fail(h, LANDAU_EUNSUPPORTED, "host-only handle");
  if (!h || !values_dev || (format != LANDAU_CSR && format != LANDAU_COO)) return fail(h, LANDAU_EINVAL, "jacobian: bad argument");
  if (!h->have_state || nbatch != h->nbatch) return fail(h, LANDAU_ESTATE, "jacobian: set_state first (batch size must match)");
  return dispatch_build(h, nbatch, values_dev, format);
});
}

int landau_jacobian(landau_t h, double *values_dev, int32_t format) {
  return guarded(h, [&]() -> int {
  if (h && h->have_state && h->nbatch != 1) return fail(h, LANDAU_ESTATE, "jacobian: state is batched");
  return landau_jacobian_batched(h, 1, values_dev, format);
});
}

// End-to-end entry: the batch is cut into K chunks; chunk c's upload (stream s_h2d), its build
// (the handle's stream) and its download (stream s_d2h) are ordered by events, so downloads of
// finished chunks overlap the builds of later ones.  Chunks are independent vertices, so the
// values are identical to one whole-batch build up to the split-j / symmetric grouping (the same
// for every chunk size at or above the symmetric threshold).
int landau_jacobian_host(landau_t h, int64_t nbatch, const double *f_host, double *values_host, int32_t format) {
  return guarded(h, [&]() -> int {
  if (h && h->host_only) return fail(h, LANDAU_EUNSUPPORTED, "host-only handle");
  if (!h || nbatch < 1 || !f_host || !values_host || (format != LANDAU_CSR && format != LANDAU_COO))
    return fail(h, LANDAU_EINVAL, "jacobian_host: bad argument");
  int rc = ensure_workspace(h, nbatch);
  if (rc) return rc;
  const int64_t nv = format == LANDAU_CSR ? h->nnz : h->ncoo;
  if (nbatch * nv > h->vals_tmp_cap) {
    drop_graphs(h);
    cudaFree(h->d_vals_tmp);
    h->d_vals_tmp = nullptr;
    CU(cudaMalloc(&h->d_vals_tmp, sizeof(double) * nbatch * nv));
    h->vals_tmp_cap = nbatch * nv;
  }
  if (!h->s_h2d) {
    CU(cudaStreamCreateWithFlags(&h->s_h2d, cudaStreamNonBlocking));
    CU(cudaStreamCreateWithFlags(&h->s_d2h, cudaStreamNonBlocking));
  }
  static const int64_t kmax = [] {
    const char *e = getenv("LANDAU_HOST_CHUNKS");
    // C4 1024 vertices (scripts/e2e_probe.py, one B200, D2H 56.7 GB/s): 8 chunks 4.65 ms, 16 4.48 ms,
    // 32 4.88 ms; a shorter first chunk (16-48 vertices) 5.0-5.9 ms
    return e ? (int64_t)atoll(e) : (int64_t)16;
  }();
  const int64_t K = std::max<int64_t>(1, std::min<int64_t>(kmax, nbatch / 32));
  std::vector<int64_t> bnd{0};   // chunk boundaries (equal chunks)
  for (int64_t c = 1; c <= K; c++) bnd.push_back(nbatch * c / K);
  while ((int64_t)h->ev_h2d.size() < K) {
    cudaEvent_t a, b;
    CU(cudaEventCreateWithFlags(&a, cudaEventDisableTiming));
    CU(cudaEventCreateWithFlags(&b, cudaEventDisableTiming));
    h->ev_h2d.push_back(a);
    h->ev_built.push_back(b);
  }
  // the copies may only start once earlier work on the handle's stream is done with the buffers
  CU(cudaEventRecord(h->ev_built[0], h->stream));
  CU(cudaStreamWaitEvent(h->s_h2d, h->ev_built[0], 0));
  CU(cudaStreamWaitEvent(h->s_d2h, h->ev_built[0], 0));
  for (int64_t c = 0; c < K; c++) {
    const int64_t b0 = bnd[c], n = bnd[c + 1] - bnd[c];
    if (n <= 0) continue;
    CU(cudaMemcpyAsync(h->d_f + b0 * h->ndof, f_host + b0 * h->ndof, sizeof(double) * n * h->ndof,
                       cudaMemcpyHostToDevice, h->s_h2d));
    CU(cudaEventRecord(h->ev_h2d[c], h->s_h2d));
    CU(cudaStreamWaitEvent(h->stream, h->ev_h2d[c], 0));
    h->fin = h->d_f + b0 * h->ndof;
    rc = dispatch_build(h, n, h->d_vals_tmp + b0 * nv, format);
    h->fin = nullptr;
    if (rc) return rc;
    CU(cudaEventRecord(h->ev_built[c], h->stream));
    CU(cudaStreamWaitEvent(h->s_d2h, h->ev_built[c], 0));
    CU(cudaMemcpyAsync(values_host + b0 * nv, h->d_vals_tmp + b0 * nv, sizeof(double) * n * nv,
                       cudaMemcpyDeviceToHost, h->s_d2h));
  }
  h->nbatch = bnd.back() - bnd[bnd.size() - 2];   // the device state now holds the last chunk's batch layout
  h->have_state = false;   // (d_f holds the whole host batch, but not as one set_state)
  CU(cudaStreamSynchronize(h->s_d2h));
  CU(cudaStreamSynchronize(h->stream));
  return LANDAU_OK;
});
}

int landau_mass(landau_t h, double shift, double *values_dev, int32_t format) {
  return guarded(h, [&]() -> int {
  if (h && h->host_only) return fail(h, LANDAU_EUNSUPPORTED, "host-only handle");
  if (!h || !values_dev || (format != LANDAU_CSR && format != LANDAU_COO)) return fail(h, LANDAU_EINVAL, "mass: bad argument");
  Timer t(h, LANDAU_T_MASS);
  ScaleCopyDesc d{};
  int64_t nmax = 0;
  for (int a = 0; a < h->S; a++) {   // every species block in one launch
    const int g = h->sgrid[a];
    d.M[a] = format == LANDAU_CSR ? h->d_mass_csr[g] : h->d_mass_coo[g];
    d.n[a] = format == LANDAU_CSR ? (int64_t)h->plan.grids[g].col.size() : h->plan.grids[g].ncoo;
    d.off[a] = format == LANDAU_CSR ? h->snnz_off[a] : h->scoo_off[a];
    d.scale[a] = shift;
    nmax = std::max(nmax, d.n[a]);
  }
  if (nmax == 0) return LANDAU_OK;
  const int blocks = (int)std::min<int64_t>((nmax + 255) / 256, 8LL * num_sms(h));
  scale_copy_species_kernel<<<dim3(blocks, h->S), 256, 0, h->stream>>>(d, values_dev);
  h->launches++;
  h->tlaunch[LANDAU_T_MASS]++;
  KCHECK();
  return LANDAU_OK;
});
}

int landau_advection(landau_t h, double Ez, double *values_dev, int32_t format) {
  return guarded(h, [&]() -> int {
  if (h && h->host_only) return fail(h, LANDAU_EUNSUPPORTED, "host-only handle");
  if (!h || !values_dev || (format != LANDAU_CSR && format != LANDAU_COO)) return fail(h, LANDAU_EINVAL, "advection: bad argument");
  Timer t(h, LANDAU_T_MASS);
  for (int a = 0; a < h->S; a++) {
    const int g = h->sgrid[a];
    const double *A = format == LANDAU_CSR ? h->d_adv_csr[g] : h->d_adv_coo[g];
    const int64_t n = format == LANDAU_CSR ? (int64_t)h->plan.grids[g].col.size() : h->plan.grids[g].ncoo;
    const int64_t off = format == LANDAU_CSR ? h->snnz_off[a] : h->scoo_off[a];
    if (n == 0) continue;
    const int blocks = (int)std::min<int64_t>((n + 255) / 256, 8LL * num_sms(h));
    scale_copy_kernel<<<blocks, 256, 0, h->stream>>>(A, Ez * h->charge[a] / h->mass[a], n, values_dev + off);
    h->launches++;
    h->tlaunch[LANDAU_T_MASS]++;
    KCHECK();
  }
  return LANDAU_OK;
});
}

int landau_point_coeffs_batched(landau_t h, int64_t nbatch, double *G_dev) {
  return guarded(h, [&]() -> int {
  if (h && h->host_only) return fail(h, LANDAU_EUNSUPPORTED, "host-only handle");
  if (!h || !G_dev) return fail(h, LANDAU_EINVAL, "point_coeffs: bad argument");
  if (!h->have_state || nbatch != h->nbatch) return fail(h, LANDAU_ESTATE, "point_coeffs: set_state first");
  int rc = dispatch_build(h, nbatch, nullptr, LANDAU_CSR);
  if (rc) return rc;
  const int64_t N = h->plan.npts;
  if (h->Nc == N) {
    CU(cudaMemcpyAsync(G_dev, h->d_G, sizeof(double) * nbatch * 5 * N, cudaMemcpyDeviceToDevice, h->stream));
  } else {
    const int64_t total = nbatch * 5 * N;
    unchunk_kernel<<<(int)std::min<int64_t>((total + 255) / 256, 4096), 256, 0, h->stream>>>(h->d_G, N, h->Nc, (int)nbatch, G_dev);
    h->launches++;
    KCHECK();
  }
  return LANDAU_OK;
});
}

int landau_point_coeffs(landau_t h, double *G_dev) {
  return guarded(h, [&]() -> int { return landau_point_coeffs_batched(h, 1, G_dev); });
}

int landau_set_timing(landau_t h, int32_t enable) {
  return guarded(h, [&]() -> int {
  if (!h) return LANDAU_EINVAL;
  for (auto &u : h->ev_used) {
    h->ev_pool.push_back(u.second.first);
    h->ev_pool.push_back(u.second.second);
  }
  h->ev_used.clear();
  for (auto &x : h->tlaunch) x = 0;
  h->timing = enable != 0;
  return LANDAU_OK;
});
}

int landau_get_timing(landau_t h, double *ms, int64_t *launches) {
  return guarded(h, [&]() -> int {
  if (h && h->host_only) return fail(h, LANDAU_EUNSUPPORTED, "host-only handle");
  if (!h) return LANDAU_EINVAL;
  CU(cudaStreamSynchronize(h->stream));
  double acc[LANDAU_NTIMERS] = {0};
  for (auto &u : h->ev_used) {
    float t = 0;
    CU(cudaEventElapsedTime(&t, u.second.first, u.second.second));
    acc[u.first] += t;
  }
  for (int i = 0; i < LANDAU_NTIMERS; i++) {
    if (ms) ms[i] = acc[i];
    if (launches) launches[i] = h->tlaunch[i];
  }
  return LANDAU_OK;
});
}

int landau_set_mirror(landau_t h, int32_t enable) {
  return guarded(h, [&]() -> int {
  if (!h) return LANDAU_EINVAL;
  if (enable < 0 || enable > 3) return fail(h, LANDAU_EINVAL, "set_mirror: mode must be 0..3");
  if (enable && !h->mirror) return fail(h, LANDAU_EUNSUPPORTED, "set_mirror: the mesh is not mirror-symmetric");
  if (enable == 3 && !h->vtx_smem) return fail(h, LANDAU_EUNSUPPORTED, "set_mirror: a vertex does not fit shared memory");
  if (h->dist_pairs && enable != 1 && enable != 2)
    return fail(h, LANDAU_EUNSUPPORTED, "set_mirror: the pair split runs the mirror slot kernel");
  if (!h->host_only) drop_graphs(h);
  h->mirror_on = enable != 0;
  h->mirror_mode = enable ? enable : 1;
  return LANDAU_OK;
});
}

int landau_set_tensor_cache(landau_t h, int32_t enable) {
  return guarded(h, [&]() -> int {
  if (!h) return LANDAU_EINVAL;
  if (h->host_only) return fail(h, LANDAU_EUNSUPPORTED, "host-only handle");
  if (!enable) {
    drop_graphs(h);
    CU(cudaStreamSynchronize(h->stream));
    cudaFree(h->d_U);
    h->d_U = nullptr;
    h->tcache = h->tcache_valid = false;
    return LANDAU_OK;
  }
  if (h->tcache) {
    if (h->tcache_recompute != (enable == 2)) drop_graphs(h);
    h->tcache_recompute = enable == 2;
    return LANDAU_OK;
  }
  const int64_t N = h->plan.npts;
  if (h->world > 1 || h->Nc != N) return fail(h, LANDAU_EUNSUPPORTED, "tensor cache needs all targets on one GPU");
  if (7 * N * N * (int64_t)sizeof(double) > (16LL << 30)) return fail(h, LANDAU_EUNSUPPORTED, "tensor cache > 16 GiB");
  if (N > INT32_MAX / 5) return fail(h, LANDAU_EUNSUPPORTED, "mesh too large for the GEMM path");
  if (!load_cublas()) return fail(h, LANDAU_EUNSUPPORTED, "cannot load libcublas.so.12");
  if (!h->cublas) {
    if (g_cublas.Create(&h->cublas)) return fail(h, LANDAU_ECUDA, "cublasCreate failed");
    if (g_cublas.SetStream(h->cublas, h->stream)) return fail(h, LANDAU_ECUDA, "cublasSetStream failed");
  }
  CU(cudaMalloc(&h->d_U, sizeof(double) * 7 * N * N));
  drop_graphs(h);
  h->tcache = true;
  h->tcache_valid = false;
  h->tcache_recompute = enable == 2;
  return LANDAU_OK;
});
}

int landau_band_info(landau_t h, int32_t grid, int32_t *bandwidth, int32_t *perm) {
  return guarded(h, [&]() -> int {
  if (!h || grid < 0 || grid >= h->plan.ngrids) return LANDAU_EINVAL;
  const GridPlan &G = h->plan.grids[grid];
  if (bandwidth) *bandwidth = G.band;
  if (perm) memcpy(perm, G.rcm_perm.data(), sizeof(int32_t) * G.ndof);
  return LANDAU_OK;
});
}

int landau_band_factor_batched(landau_t h, int64_t nbatch, double shift, const double *J_csr_dev) {
  return guarded(h, [&]() -> int {
  return landau_band_factor_field_batched(h, nbatch, shift, 0.0, J_csr_dev);
});
}

// The band factorisation; with rhs (the implicit step, DMMA kernel only) the kernel also eliminates rhs
// forward into d_yfwd and writes only the U part of the factor (band_fwd_done: only the backward pass of
// the solve remains, see band_solve_impl).  Returns LANDAU_EUNSUPPORTED (nothing launched) when rhs is
// given and the DMMA kernel does not apply.
int band_factor_impl(landau_t h, int64_t nbatch, double shift, double Ez, const double *J_csr_dev, const double *rhs) {
  if (h && h->host_only) return fail(h, LANDAU_EUNSUPPORTED, "host-only handle");
  if (!h || nbatch < 1 || !J_csr_dev) return fail(h, LANDAU_EINVAL, "band_factor: bad argument");
  int maxPp = 8, maxn = 0, maxent = 0;
  for (auto &d : h->band_desc) {
    maxPp = std::max(maxPp, d.Pp);
    maxn = std::max(maxn, d.n);
    maxent = std::max(maxent, d.nent);
  }
  // one CTA per matrix with the active window in registers: vertex-grid sizes (C1-C4); a single large
  // grid (C5) would need a multi-CTA factorisation (not built)
  if (maxPp > kBandMaxP) return fail(h, LANDAU_EUNSUPPORTED, "band factor: half-bandwidth above 127");
  // band_lu2_kernel's shared memory: pivot rows/columns (double-buffered, padded), 3 x 8 dense
  // entering rows of 4P, the entry lists
  const size_t smem = sizeof(double) * (2 * (2 * maxPp + 2 * (maxPp / 8 * 10) + 8) + 24 * 4 * maxPp) +
                      sizeof(int32_t) * (maxn + 1) + sizeof(uint16_t) * maxent;
  if (smem > 200 * 1024) return fail(h, LANDAU_EUNSUPPORTED, "band factor: grid too large for one CTA");
  if (nbatch > h->band_cap) {
    cudaFree(h->d_band);
    cudaFree(h->d_Aent);
    h->d_band = h->d_Aent = nullptr;
    CU(cudaMalloc(&h->d_band, sizeof(double) * nbatch * h->band_bstride));
    CU(cudaMalloc(&h->d_Aent, sizeof(double) * nbatch * std::max<int64_t>(h->ent_bstride, 1)));
    h->band_cap = nbatch;
  }
  Timer t(h, LANDAU_T_FACTOR);
  for (int a = 0; a < h->S; a++) {
    const int g = h->sgrid[a];
    const int64_t nent = h->band_desc[a].nent;
    if (!nent) continue;
    const int blocks = (int)std::min<int64_t>((nent * nbatch + 255) / 256, 16LL * num_sms(h));
    band_gather_kernel<<<blocks, 256, 0, h->stream>>>(nent, h->d_ent_slot[g], h->d_mass_csr[g], h->d_adv_csr[g],
                                                      Ez * h->charge[a] / h->mass[a], J_csr_dev, h->nnz,
                                                      h->snnz_off[a], shift, h->d_Aent, h->ent_bstride,
                                                      h->band_desc[a].aoff, (int)nbatch);
    h->launches++;
    KCHECK();
  }
  // threads: the tile owners, the 2B + 1 factor-row writers, and enough to stage one group's entering
  // entries kBandE per thread (threads past the tiles own none and only stage and write)
  const int tiles_lu = (maxPp / (maxPp <= 88 ? 4 : 8)) * (maxPp / 8);
  const int stage_lu = (h->band_ent_max + kBandE - 1) / kBandE;
  const int threads_lu = std::min(256, std::max(64, (std::max(std::max(tiles_lu, 2 * maxPp - 1), stage_lu) + 31) / 32 * 32));
  if (h->band_ent_max > kBandE * threads_lu) return fail(h, LANDAU_EUNSUPPORTED, "band factor: too many entries per row group");
  const unsigned grid = (unsigned)(nbatch * h->S);
  static const int band_minb = [] {
    const char *e = getenv("LANDAU_BAND_MINB");
    return e ? atoi(e) : 2;
  }();
  static const bool band_cw = [] {   // opt-in: the column-warp kernel measured slower
    const char *e = getenv("LANDAU_BAND_CW");
    return e && atoi(e) != 0;
  }();
  const void *kfn;
  size_t ksmem = smem;
  unsigned threads = (unsigned)threads_lu;
  bool same_p = true;
  for (auto &d : h->band_desc) same_p = same_p && d.Pp == maxPp;
  static const void *const cw_kernels[12] = {
      (const void *)band_lu_cw_kernel<1>, (const void *)band_lu_cw_kernel<2>,  (const void *)band_lu_cw_kernel<3>,
      (const void *)band_lu_cw_kernel<4>, (const void *)band_lu_cw_kernel<5>,  (const void *)band_lu_cw_kernel<6>,
      (const void *)band_lu_cw_kernel<7>, (const void *)band_lu_cw_kernel<8>,  (const void *)band_lu_cw_kernel<9>,
      (const void *)band_lu_cw_kernel<10>, (const void *)band_lu_cw_kernel<11>, (const void *)band_lu_cw_kernel<12>};
  static const bool band_mma = [] {   // the blocked DMMA factorisation (kernels_band_mma.cuh)
    const char *e = getenv("LANDAU_BAND_MMA");
    return !(e && atoi(e) == 0);
  }();
#define BM(NT) (const void *)band_lu_mma_kernel<NT, false>
#define BF(NT) (const void *)band_lu_mma_kernel<NT, true>
  static const void *const mma_kernels[18] = {nullptr, nullptr, nullptr, BM(3),  BM(4),  BM(5),  BM(6),  BM(7),  BM(8),
                                              BM(9),   BM(10),  BM(11),  BM(12), BM(13), BM(14), BM(15), BM(16), BM(17)};
  static const void *const mma_kernels_fwd[18] = {nullptr, nullptr, nullptr, BF(3),  BF(4),  BF(5),  BF(6),
                                                  BF(7),   BF(8),   BF(9),   BF(10), BF(11), BF(12), BF(13),
                                                  BF(14),  BF(15),  BF(16),  BF(17)};
#undef BM
#undef BF
  const int mma_nt = maxPp / 8 + 1;
  // the DMMA kernel applies to every species block (window NT = P/8 + 1 tiles per side, 3..17); blocks
  // of different bandwidth (separate grids, C3) are factored by one launch per species
  bool mma_all = band_mma && h->band_ent_max <= kBmE * 32 * kBmWarps;
  for (auto &d : h->band_desc) mma_all = mma_all && d.Pp % 8 == 0 && d.Pp / 8 + 1 >= 3 && d.Pp / 8 + 1 <= 17;
  const bool mma_ok = mma_all && same_p;
  if (rhs && (band_cw || !mma_all)) return LANDAU_EUNSUPPORTED;
  if (rhs && nbatch > h->yfwd_cap) {
    cudaFree(h->d_yfwd);
    h->d_yfwd = nullptr;
    CU(cudaMalloc(&h->d_yfwd, sizeof(double) * nbatch * std::max<int64_t>(h->ndof, 1)));
    h->yfwd_cap = nbatch;
  }
  static const bool per_species = [] {   // test knob: the per-species launches even for equal bands
    const char *e = getenv("LANDAU_BAND_PER_SPECIES");
    return e && atoi(e) != 0;
  }();
  if (mma_all && (!same_p || per_species) && !band_cw) {   // one DMMA launch per species block (its own window)
    for (int a = 0; a < h->S; a++) {
      const int nt = h->band_desc[a].Pp / 8 + 1;
      const void *kf = rhs ? mma_kernels_fwd[nt] : mma_kernels[nt];
      const size_t sm = sizeof(double) * (band_mma_smem_doubles(nt) + (rhs ? h->band_desc[a].n : 0));
      if (sm > 200 * 1024) return fail(h, LANDAU_EUNSUPPORTED, "band factor: grid too large for one CTA");
      if (sm > 48 * 1024) CU(cudaFuncSetAttribute(kf, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm));
      const double *a0 = h->d_Aent;
      int64_t a1 = h->ent_bstride;
      double *a2 = h->d_band;
      int64_t a3 = h->band_bstride;
      const BandDesc *a4 = h->d_band_desc + a;   // nsp = 1: this block only
      int a5 = 1;
      const double *a6 = rhs;
      double *a7 = h->d_yfwd;
      const int32_t *a8 = h->d_perm_all;
      const int64_t *a9 = h->d_perm_off + a, *a10 = h->d_vec_off + a;
      int64_t a11 = h->ndof;
      void *args[] = {&a0, &a1, &a2, &a3, &a4, &a5, &a6, &a7, &a8, &a9, &a10, &a11};
      CU(cudaLaunchKernel(kf, dim3((unsigned)nbatch), dim3(32 * kBmWarps), args, sm, h->stream));
      h->launches++;
      KCHECK();
    }
    h->tlaunch[LANDAU_T_FACTOR]++;
    h->band_nbatch = nbatch;
    h->band_fwd_done = rhs != nullptr;
    return LANDAU_OK;
  }
  if (band_cw && same_p && maxPp <= 96 && maxPp % 8 == 0 && h->band_ent_max <= kBandE * 256) {
    // column-warp kernel with look-ahead: 8 warps of P / 8 columns (one window width per launch)
    kfn = cw_kernels[maxPp / 8 - 1];
    ksmem = sizeof(double) * (2 * kCwRing + 48) * maxPp;
    threads = 256;
  } else if (mma_ok) {
    // blocked factorisation, DMMA trailing updates (kernels_band_mma.cuh): C4 2.0 ms vs 3.2 ms
    kfn = rhs ? mma_kernels_fwd[mma_nt] : mma_kernels[mma_nt];
    ksmem = sizeof(double) * (band_mma_smem_doubles(mma_nt) + (rhs ? maxn : 0));
    threads = 32 * kBmWarps;
  } else if (maxPp <= 88)   // 4 x 8 tiles, <= 242 threads; two CTAs per SM (128 registers) or one
    kfn = band_minb >= 2 ? (const void *)band_lu2_kernel<4, 8, 2> : (const void *)band_lu2_kernel<4, 8, 1>;
  else               // 8 x 8 tiles, <= 256 threads
    kfn = (const void *)band_lu2_kernel<8, 8, 1>;
  if (ksmem > 200 * 1024) return fail(h, LANDAU_EUNSUPPORTED, "band factor: grid too large for one CTA");
  if (ksmem > 48 * 1024) CU(cudaFuncSetAttribute(kfn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)ksmem));
  {
    const double *a0 = h->d_Aent;
    int64_t a1 = h->ent_bstride;
    double *a2 = h->d_band;
    int64_t a3 = h->band_bstride;
    const BandDesc *a4 = h->d_band_desc;
    int a5 = h->S;
    const double *a6 = rhs;
    double *a7 = h->d_yfwd;
    const int32_t *a8 = h->d_perm_all;
    const int64_t *a9 = h->d_perm_off, *a10 = h->d_vec_off;
    int64_t a11 = h->ndof;
    void *args[] = {&a0, &a1, &a2, &a3, &a4, &a5, &a6, &a7, &a8, &a9, &a10, &a11};
    // (the register-tile and column-warp kernels take the first six arguments)
    CU(cudaLaunchKernel(kfn, dim3(grid), dim3(threads), args, ksmem, h->stream));
  }
  h->launches++;
  h->tlaunch[LANDAU_T_FACTOR]++;
  KCHECK();
  h->band_nbatch = nbatch;
  h->band_fwd_done = rhs != nullptr;
  return LANDAU_OK;
}

int landau_band_factor_field_batched(landau_t h, int64_t nbatch, double shift, double Ez, const double *J_csr_dev) {
  return guarded(h, [&]() -> int { return band_factor_impl(h, nbatch, shift, Ez, J_csr_dev, nullptr); });
}

// yfwd: the fused factorisation's forward-eliminated rhs (backward pass only); else b_dev is solved fully
int band_solve_impl(landau_t h, int64_t nbatch, const double *b_dev, double *x_dev, const double *yfwd) {
  if (h && h->host_only) return fail(h, LANDAU_EUNSUPPORTED, "host-only handle");
  if (!h || nbatch < 1 || (!b_dev && !yfwd) || !x_dev) return fail(h, LANDAU_EINVAL, "band_solve: bad argument");
  if (h->band_nbatch != nbatch) return fail(h, LANDAU_ESTATE, "band_solve: factor this batch first");
  if (h->band_fwd_done != (yfwd != nullptr))
    return fail(h, LANDAU_ESTATE, "band_solve: the last factorisation was the implicit step's fused one; factor again");
  Timer t(h, LANDAU_T_SOLVE);
  int maxn = 0, maxB = 0;
  for (auto &d : h->band_desc) maxn = std::max(maxn, d.n), maxB = std::max(maxB, d.B);
  constexpr int kWarps = 4;
  const size_t smem = sizeof(double) * kWarps * (maxn + maxB + 1 + (kBandD + 1) * (maxB + 1));
  if (smem > 48 * 1024) CU(cudaFuncSetAttribute(band_solve_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  const int64_t warps = nbatch * h->S;
  band_solve_kernel<<<(unsigned)((warps + kWarps - 1) / kWarps), 32 * kWarps, smem, h->stream>>>(
      h->d_band, h->band_bstride, h->d_band_desc, h->d_perm_all, h->d_perm_off, h->d_vec_off, h->ndof, maxn, maxB,
      b_dev, x_dev, h->S, (int)nbatch, yfwd);
  h->launches++;
  h->tlaunch[LANDAU_T_SOLVE]++;
  KCHECK();
  return LANDAU_OK;
}

int landau_band_solve_batched(landau_t h, int64_t nbatch, const double *b_dev, double *x_dev) {
  return guarded(h, [&]() -> int { return band_solve_impl(h, nbatch, b_dev, x_dev, nullptr); });
}

int landau_implicit_step_batched(landau_t h, int64_t nbatch, double dt, double Ez, const double *f_old_dev,
                                 double *f_new_dev, int32_t max_iter, double rtol, int32_t *iters, double *dnorm) {
  return landau_implicit_step_source_batched(h, nbatch, dt, Ez, f_old_dev, nullptr, f_new_dev, max_iter, rtol, iters,
                                             dnorm);
}

int landau_implicit_step_source_batched(landau_t h, int64_t nbatch, double dt, double Ez, const double *f_old_dev,
                                        const double *src_dev, double *f_new_dev, int32_t max_iter, double rtol,
                                        int32_t *iters, double *dnorm) {
  return guarded(h, [&]() -> int {
  if (h && h->host_only) return fail(h, LANDAU_EUNSUPPORTED, "host-only handle");
  if (!h || nbatch < 1 || !f_old_dev || !f_new_dev || f_old_dev == f_new_dev || max_iter < 1 || !(dt > 0))
    return fail(h, LANDAU_EINVAL, "implicit_step: bad argument");
  if (nbatch > h->step_cap) {
    cudaFree(h->d_Jwork);
    cudaFree(h->d_rhs);
    cudaFree(h->d_norms);
    if (h->h_norms) cudaFreeHost(h->h_norms);
    h->d_Jwork = h->d_rhs = h->d_norms = h->h_norms = nullptr;
    CU(cudaMalloc(&h->d_Jwork, sizeof(double) * nbatch * std::max<int64_t>(h->nnz, 1)));
    CU(cudaMalloc(&h->d_rhs, sizeof(double) * nbatch * std::max<int64_t>(h->ndof, 1)));
    CU(cudaMalloc(&h->d_norms, sizeof(double) * 2 * nbatch));
    CU(cudaMallocHost(&h->h_norms, sizeof(double) * 2 * nbatch));
    cudaFree(h->d_srcx);
    h->d_srcx = nullptr;
    CU(cudaMalloc(&h->d_srcx, sizeof(double) * nbatch * std::max<int64_t>(h->ndof, 1)));
    h->step_cap = nbatch;
  }
  // rhs = M f_old / dt (species blocks) or, with a source, M (f_old / dt + sigma) (Eq. 4's (psi, S_a) =
  // M sigma, R-7); initial iterate f_old
  const double *xin = f_old_dev;
  double rscale = 1.0 / dt;
  if (src_dev) {
    const int64_t n = nbatch * h->ndof;
    axpby_kernel<<<(unsigned)std::min<int64_t>((n + 255) / 256, 16LL * num_sms(h)), 256, 0, h->stream>>>(
        n, 1.0 / dt, f_old_dev, src_dev, h->d_srcx);
    h->launches++;
    KCHECK();
    xin = h->d_srcx;
    rscale = 1.0;
  }
  for (int a = 0; a < h->S; a++) {
    const int g = h->sgrid[a];
    const int n = h->plan.grids[g].ndof;
    if (!n) continue;
    const int64_t warps = nbatch * n;
    block_spmv_kernel<<<(unsigned)((warps * 32 + 255) / 256), 256, 0, h->stream>>>(
        h->d_rowptr[g], h->d_col[g], h->d_mass_csr[g], n, h->soff[a], h->ndof, rscale, xin, h->d_rhs,
        (int)nbatch);
    h->launches++;
    KCHECK();
  }
  CU(cudaMemcpyAsync(f_new_dev, f_old_dev, sizeof(double) * nbatch * h->ndof, cudaMemcpyDeviceToDevice, h->stream));
  int it = 0;
  double worst = 0.0;
  for (it = 1; it <= max_iter; it++) {
    // quasi-Newton iteration (@10500-10978): J about the current iterate, then
    // (M/dt + E_z (e/m) A_E - J(f^k)) f^{k+1} = M f_old / dt  by the band LU
    int rc = landau_set_state_batched(h, nbatch, f_new_dev);
    if (!rc) rc = dispatch_build(h, nbatch, h->d_Jwork, LANDAU_CSR);
    // the fused factorisation (rhs eliminated forward inside the DMMA kernel, U stored alone) where it
    // applies (LANDAU_BAND_FUSED=0: factor + full solve)
    static const bool fused = [] {
      const char *e = getenv("LANDAU_BAND_FUSED");
      return !(e && atoi(e) == 0);
    }();
    if (!rc) {
      const int rf = fused ? band_factor_impl(h, nbatch, 1.0 / dt, Ez, h->d_Jwork, h->d_rhs) : LANDAU_EUNSUPPORTED;
      if (rf == LANDAU_OK) {
        rc = band_solve_impl(h, nbatch, nullptr, f_new_dev, h->d_yfwd);
      } else if (rf == LANDAU_EUNSUPPORTED) {
        rc = band_factor_impl(h, nbatch, 1.0 / dt, Ez, h->d_Jwork, nullptr);
        if (!rc) rc = band_solve_impl(h, nbatch, h->d_rhs, f_new_dev, nullptr);
      } else {
        rc = rf;
      }
    }
    if (rc) return rc;
    delta_norm_kernel<<<(unsigned)nbatch, 256, 0, h->stream>>>(f_new_dev, h->d_f, h->ndof, h->d_norms);
    h->launches++;
    KCHECK();
    if (rtol > 0 || it == max_iter) {
      CU(cudaMemcpyAsync(h->h_norms, h->d_norms, sizeof(double) * 2 * nbatch, cudaMemcpyDeviceToHost, h->stream));
      CU(cudaStreamSynchronize(h->stream));
      worst = 0.0;
      for (int64_t b = 0; b < nbatch; b++)
        worst = std::max(worst, std::sqrt(h->h_norms[2 * b] / std::max(h->h_norms[2 * b + 1], 1e-300)));
      if (rtol > 0 && worst <= rtol) break;
    }
  }
  if (iters) *iters = std::min(it, (int)max_iter);
  if (dnorm) *dnorm = worst;
  return LANDAU_OK;
});
}

int landau_get_vtx_schedule(landau_t h, int32_t *nrounds, int32_t *weight_prefix, int32_t *ctas) {
  return guarded(h, [&]() -> int {
  if (!h) return LANDAU_EINVAL;
  if (!h->vtx_smem) return fail(h, LANDAU_EUNSUPPORTED, "vtx schedule: the per-vertex kernel is not available");
  if (nrounds) *nrounds = h->nvtx_rounds;
  if (weight_prefix) {
    if (h->host_only) return fail(h, LANDAU_EUNSUPPORTED, "host-only handle");
    CU(cudaMemcpy(weight_prefix, h->d_vtx_wp, sizeof(int32_t) * (h->nvtx_rounds + 1), cudaMemcpyDeviceToHost));
  }
  if (ctas) *ctas = h->host_only ? 0 : num_sms(h) * kVtxMinB;
  return LANDAU_OK;
});
}

int landau_get_vtx_split(landau_t h, int64_t nbatch, int32_t *first_cta, int32_t *last_cta) {
  return guarded(h, [&]() -> int {
  if (!h || nbatch < 1 || !first_cta || !last_cta) return fail(h, LANDAU_EINVAL, "vtx split: bad argument");
  if (!h->vtx_smem) return fail(h, LANDAU_EUNSUPPORTED, "vtx schedule: the per-vertex kernel is not available");
  const int S = h->host_only ? 148 * kVtxMinB : num_sms(h) * kVtxMinB;
  std::vector<int16_t> ord;
  std::vector<int32_t> wpv;
  vtx_tables(h, nbatch, S, ord, wpv);
  const int R = h->nvtx_rounds;
  const int64_t Wtot = nbatch * h->vtx_Wv;
  for (int64_t v = 0; v < nbatch; v++) {
    const int32_t *w = wpv.data() + v * (R + 1);
    first_cta[v] = (int32_t)(((v * h->vtx_Wv + w[0]) * S) / Wtot);
    last_cta[v] = (int32_t)(((v * h->vtx_Wv + w[R - 1]) * S) / Wtot);
  }
  return LANDAU_OK;
});
}

int landau_get_mirror(landau_t h, int32_t *mirror_symmetric, int32_t *mirror_active) {
  return guarded(h, [&]() -> int {
  if (!h) return LANDAU_EINVAL;
  if (mirror_symmetric) *mirror_symmetric = h->mirror_sym ? 1 : 0;
  if (mirror_active) *mirror_active = (h->mirror && h->mirror_on) ? 1 : 0;
  return LANDAU_OK;
});
}

int landau_get_stats(landau_t h, landau_stats_t *stats) {
  return guarded(h, [&]() -> int {
  if (!h || !stats) return LANDAU_EINVAL;
  *stats = h->stats;
  return LANDAU_OK;
});
}

int landau_get_launch_count(landau_t h, int64_t *count) {
  return guarded(h, [&]() -> int {
  if (!h || !count) return LANDAU_EINVAL;
  *count = h->launches;
  return LANDAU_OK;
});
}

}  // extern "C"

static int create_impl(landau_t &h, landau_t *out, const landau_mesh_t *mesh, const landau_params_t *prm, int32_t cuda_device,
                void *cuda_stream, const landau_dist_t *dist) {
  if (!out || !mesh || !prm) return fail(h, LANDAU_EINVAL, "null argument");
  *out = nullptr;
  if (mesh->ngrids < 1 || mesh->ngrids > kMaxSpecies || !mesh->ncells || !mesh->cells || !mesh->radius)
    return fail(h, LANDAU_EINVAL, "bad mesh descriptor");
  if (prm->order < 2 || prm->order > 4) return fail(h, LANDAU_EINVAL, "order must be 2, 3 or 4");
  if (prm->nq1d != 0 && prm->nq1d != prm->order + 1) return fail(h, LANDAU_EUNSUPPORTED, "nq1d must be 0 or order+1");
  if (prm->nspecies < 1 || prm->nspecies > kMaxSpecies || !prm->mass || !prm->charge || !prm->grid)
    return fail(h, LANDAU_EINVAL, "bad species descriptor");
  for (int a = 0; a < prm->nspecies; a++)
    if (!(prm->mass[a] > 0) || prm->grid[a] < 0 || prm->grid[a] >= mesh->ngrids || !std::isfinite(prm->charge[a]))
      return fail(h, LANDAU_EINVAL, "bad species " + std::to_string(a));
  int rank = 0, world = 1, mode = LANDAU_DIST_REPLICATE;
  if (dist) {
    rank = dist->rank;
    world = dist->world;
    mode = dist->mode;
    if (world < 1 || rank < 0 || rank >= world || mode < 0 || mode > 2) return fail(h, LANDAU_EINVAL, "bad dist descriptor");
    if (mode != LANDAU_DIST_ELEMENTS) world = 1, rank = 0;   // replicas / caller-split batches: independent handles
  }
  h = new landau_s();
  h->device = cuda_device;
  h->stream = (cudaStream_t)cuda_stream;
  if (const char *e = getenv("LANDAU_GRAPHS")) h->use_graphs = atoi(e) != 0;
  h->rank = rank;
  h->world = world;
  h->mode = mode;
  std::string msg = build_plan(mesh->ngrids, mesh->ncells, mesh->cells, mesh->radius, prm->order, h->plan);
  if (!msg.empty()) {
    delete h;
    h = nullptr;
    return fail(nullptr, LANDAU_EINVAL, msg);
  }
  const Plan &P = h->plan;
  h->S = prm->nspecies;
  h->nu = prm->nu;
  h->spc = SpeciesConst{};
  h->spc.nspecies = h->S;
  h->spc.ngrids = P.ngrids;
  h->soff.assign(h->S + 1, 0);
  h->snnz_off.assign(h->S + 1, 0);
  h->scoo_off.assign(h->S + 1, 0);
  for (int a = 0; a < h->S; a++) {
    const int g = prm->grid[a];
    h->mass.push_back(prm->mass[a]);
    h->charge.push_back(prm->charge[a]);
    h->sgrid.push_back(g);
    const double e2 = prm->charge[a] * prm->charge[a], im = 1.0 / prm->mass[a];
    h->spc.e2[a] = e2;
    h->spc.e2m[a] = e2 * im;
    h->spc.fD[a] = -prm->nu * e2 * im * im;
    h->spc.fK[a] = prm->nu * e2 * im;
    h->spc.grid_sp[g][h->spc.grid_nsp[g]++] = a;
    h->soff[a + 1] = h->soff[a] + P.grids[g].ndof;
    h->snnz_off[a + 1] = h->snnz_off[a] + (int64_t)P.grids[g].col.size();
    h->scoo_off[a + 1] = h->scoo_off[a] + P.grids[g].ncoo;
    h->spc.soff[a] = h->soff[a];
  }
  h->ndof = h->soff[h->S];
  h->nnz = h->snnz_off[h->S];
  h->ncoo = h->scoo_off[h->S];
  // element partition
  landau_partition(P.ncell, world, rank, &h->e0, &h->e1);
  h->chunk_cells = (P.ncell + world - 1) / world;
  h->Nc = mode == LANDAU_DIST_ELEMENTS ? h->chunk_cells * P.nqp : P.npts;
  int rc;
  h->mirror_sym = detect_mirror(P, h->mir_pu, h->mir_pm);
  if (cuda_device == LANDAU_HOST_ONLY) {
    h->host_only = true;
    *out = h;
    return LANDAU_OK;
  }
  (void)cudaGetLastError();   // a non-sticky error left by other code (a library, a freed handle) is not ours
  cudaError_t ce = cudaSetDevice(cuda_device);
  if (ce != cudaSuccess) {
    std::string m = std::string("cudaSetDevice: ") + cudaGetErrorString(ce);
    delete h;
    h = nullptr;
    return fail(nullptr, LANDAU_ECUDA, m);
  }
  auto bail = [&](int code) {
    std::string m = h->err;
    landau_destroy(h);
    h = nullptr;
    return fail(nullptr, code, m);
  };
  if ((rc = upload(h, &h->d_r, P.pr)) || (rc = upload(h, &h->d_z, P.pz)) || (rc = upload(h, &h->d_w, P.pw)) ||
      (rc = upload(h, &h->d_h, P.cell_h)) || (rc = upload(h, &h->d_cell_grid, P.cell_grid)) ||
      (rc = upload(h, &h->d_ext_ptr, P.ext_ptr)) || (rc = upload(h, &h->d_ext_dof, P.ext_dof)) ||
      (rc = upload(h, &h->d_ext_w, P.ext_w)))
    return bail(rc);
  {
    std::vector<double> tab(P.tab_phi);
    tab.insert(tab.end(), P.tab_dxi.begin(), P.tab_dxi.end());
    tab.insert(tab.end(), P.tab_deta.begin(), P.tab_deta.end());
    tab.insert(tab.end(), P.tab1_L.begin(), P.tab1_L.end());   // at 3 NB^2: 1-D factors (element_sf_kernel)
    tab.insert(tab.end(), P.tab1_D.begin(), P.tab1_D.end());
    if ((rc = upload(h, &h->d_tab, tab))) return bail(rc);
  }
  {   // do two distinct points share their coordinates (only possible across grids)?
    std::vector<std::pair<double, double>> rz(P.npts);
    for (int64_t i = 0; i < P.npts; i++) rz[i] = {P.pr[i], P.pz[i]};
    std::sort(rz.begin(), rz.end());
    for (int64_t i = 1; i < P.npts; i++)
      if (rz[i] == rz[i - 1]) h->coincident = true;
  }
  if (world == 1) {   // work items + slot map of the symmetric inner kernel
    const int T = (int)((P.npts + 31) / 32);
    std::vector<SymItem> items;
    std::vector<std::vector<int32_t>> slots_of(T);
    int slot = 0;
    for (int b = 0; b < T; b++) {          // column b: the diagonal, then i-tiles a < b, kSymNI at a time
      items.push_back({{b, -1, -1}, b, 0, slot});
      slots_of[b].push_back(slot);
      slots_of[b].push_back(slot + 1);
      slot += 2;
      for (int a = 0; a < b; a += kSymNI) {
        SymItem it{{-1, -1, -1}, b, std::min(kSymNI, b - a), slot};
        for (int t = 0; t < it.n; t++) {
          it.a[t] = a + t;
          slots_of[a + t].push_back(slot++);
        }
        slots_of[b].push_back(slot++);
        items.push_back(it);
      }
    }
    std::vector<int32_t> tptr(1, 0), tslots;
    for (int t = 0; t < T; t++) {
      tslots.insert(tslots.end(), slots_of[t].begin(), slots_of[t].end());
      tptr.push_back((int32_t)tslots.size());
    }
    h->ntiles = T;
    h->nsym_items = (int64_t)items.size();
    h->nsym_slots = slot;
    if ((rc = upload(h, &h->d_sym_items, items)) || (rc = upload(h, &h->d_tile_ptr, tptr)) ||
        (rc = upload(h, &h->d_tile_slots, tslots)))
      return bail(rc);
  }
  // mirror symmetry z -> -z of every grid (inner_mir_kernel); with several ranks (element split) the
  // tile pairs are split over the ranks and the partial G summed by one all-reduce (pair split)
  if ((world == 1 || mode == LANDAU_DIST_ELEMENTS) && mirror_enabled()) {
    const std::vector<int32_t> &pu = h->mir_pu, &pm = h->mir_pm;
    std::vector<double> rU, zU;
    const bool ok = h->mirror_sym;
    for (size_t k = 0; k < pu.size(); k++) {
      rU.push_back(P.pr[pu[k]]);
      zU.push_back(P.pz[pu[k]]);   // the mirror pm[k] sits at exactly (r, -z) (bit-exact, detect_mirror)
    }
    if (ok && !pu.empty()) {
      const int64_t H = (int64_t)pu.size();
      const int T = (int)((H + 31) / 32);
      // slot-kernel items: every tile pair (a <= b) once, U and V together, as runs of up to `run`
      // consecutive i-tiles a0 .. a0+na-1 < b against one j-tile b (slots: na forward, then one
      // reverse), and the diagonal items (b, b) (slots: forward, reverse); two sets (run 1 and
      // LANDAU_MIR_RUN).  world > 1: this rank's share of the pairs (landau_pair_partition), local slots
      static const int mir_run = [] {
        const char *e = getenv("LANDAU_MIR_RUN");
        const int v = e ? atoi(e) : 4;
        return v < 1 ? 1 : v;
      }();
      int64_t iq0 = 0, iq1 = (int64_t)T * (T + 1) / 2;
      if (world > 1) landau_pair_partition(T, world, rank, &iq0, &iq1);
      if (world == 1)
        if (const char *e = getenv("LANDAU_PAIR_SPLIT_EMULATE")) {   // test hook: "world:rank" -- this
          int ew = 1, er = 0;                                         // rank's items only, no all-reduce
          if (sscanf(e, "%d:%d", &ew, &er) == 2 && ew >= 1 && er >= 0 && er < ew) landau_pair_partition(T, ew, er, &iq0, &iq1);
        }
      for (int set = 0; set < 2; set++) {
        const int run = set == 0 ? 1 : mir_run;
        if (set == 1 && run == 1) break;
        std::vector<int4> items;
        std::vector<std::vector<int32_t>> slots_of(T);
        int slot = 0;
        int64_t qg = 0;
        for (int b = 0; b < T; b++) {
          int run0 = -1, runn = 0;
          auto flush = [&]() {
            if (!runn) return;
            items.push_back(make_int4(run0, runn, b, slot));
            for (int t = 0; t < runn; t++) slots_of[run0 + t].push_back(slot++);
            slots_of[b].push_back(slot++);
            runn = 0;
          };
          for (int a = 0; a <= b; a++, qg++) {
            if (qg < iq0 || qg >= iq1) continue;
            if (a == b) {
              flush();
              items.push_back(make_int4(b, 0, b, slot));
              slots_of[b].push_back(slot++);
              slots_of[b].push_back(slot++);
              continue;
            }
            if (runn && (a != run0 + runn || runn == run)) flush();
            if (!runn) run0 = a;
            runn++;
          }
          flush();
        }
        std::vector<int32_t> tptr(1, 0), tslots;
        for (int t = 0; t < T; t++) {
          tslots.insert(tslots.end(), slots_of[t].begin(), slots_of[t].end());
          tptr.push_back((int32_t)tslots.size());
        }
        auto &ms = h->mset[set];
        ms.nitems = (int64_t)items.size();
        ms.nslots = slot;
        if (set == 0)
          for (const int4 &it : items) h->mir_evals += it.y == 0 ? 33 * 32 : (int64_t)it.y * 2 * 32 * 32;
        if ((rc = upload(h, &ms.items, items)) || (rc = upload(h, &ms.tile_ptr, tptr)) ||
            (rc = upload(h, &ms.tile_slots, tslots)))
          return bail(rc);
      }
      // per-vertex kernel schedule: round-robin tournament of the T tiles (circle method; rounds of
      // disjoint tile pairs), then the diagonal items in rounds of kVtxWarps.  For odd T every round
      // leaves one tile out (the bye); when the CTA has a warp to spare for it ((T + 1)/2 <=
      // kVtxWarps), the bye tile's diagonal item joins that round (last, for the spare warp) and no
      // diagonal rounds remain.
      std::vector<VtxItem> vitems;
      std::vector<int32_t> vround(1, 0);
      {
        const int Tp = T + (T & 1);
        const bool bye_diag = (T & 1) && (T + 1) / 2 <= kVtxWarps;
        for (int rd = 0; rd + 1 < Tp; rd++) {
          int bye = -1;
          for (int q = 0; q < Tp / 2; q++) {
            const int x = q == 0 ? Tp - 1 : (rd + q) % (Tp - 1);
            const int y = q == 0 ? rd : (rd - q + Tp - 1) % (Tp - 1);
            if (x < T && y < T) vitems.push_back({std::min(x, y), std::max(x, y)});
            else bye = x < T ? x : y;
          }
          if (bye_diag && bye >= 0) vitems.push_back({bye, bye});
          if ((int)vitems.size() > vround.back()) vround.push_back((int32_t)vitems.size());
        }
        if (!bye_diag)
          for (int t = 0; t < T; t++) {
            vitems.push_back({t, t});
            if ((t + 1) % kVtxWarps == 0 || t + 1 == T) vround.push_back((int32_t)vitems.size());
          }
      }
      const size_t vsmem = vtx_smem_bytes((int64_t)T * 32);
      h->vtx_smem = world == 1 && vsmem <= (size_t)200 * 1024 && T >= 2 && (int)vround.size() - 1 <= kVtxMaxRounds ? vsmem : 0;
      h->nvtx_rounds = (int)vround.size() - 1;
      // stream-K weights: a round lasts as long as its longest item (pair item 2, diagonal item 1)
      std::vector<int32_t> vwp(1, 0);
      for (int rd = 0; rd < h->nvtx_rounds; rd++) {
        int w = 1;
        for (int q = vround[rd]; q < vround[rd + 1]; q++) w = std::max(w, vitems[q].a == vitems[q].b ? 1 : 2);
        vwp.push_back(vwp.back() + w);
      }
      h->vtx_Wv = vwp.back();
      h->vtx_w.clear();
      for (int rd = 0; rd < h->nvtx_rounds; rd++) h->vtx_w.push_back(vwp[rd + 1] - vwp[rd]);
      if (h->vtx_smem) {
        if ((rc = upload(h, &h->d_vtx_items, vitems)) || (rc = upload(h, &h->d_vtx_round_ptr, vround)) ||
            (rc = upload(h, &h->d_vtx_wp, vwp)))
          return bail(rc);
        if (!h->host_only) {
          if (!raise_vtx_smem_attr(cuda_device, vsmem)) return bail(fail(h, LANDAU_ECUDA, "inner_vtx_kernel smem attribute"));
        }
      }
      h->mirror = true;
      h->H = H;
      // inverse mirror map: point -> upper-half index ut, + H when the point is the mirror pm[ut]
      std::vector<int32_t> pinv(P.npts, -1);
      for (int64_t u = 0; u < H; u++) {
        pinv[pu[u]] = (int32_t)u;
        pinv[pm[u]] = (int32_t)(u + H);
      }
      if ((rc = upload(h, &h->d_rU, rU)) || (rc = upload(h, &h->d_zU, zU)) || (rc = upload(h, &h->d_pu, pu)) ||
          (rc = upload(h, &h->d_pm, pm)) || (rc = upload(h, &h->d_pinv, pinv)))
        return bail(rc);
      if (world > 1) {   // pair split: every rank targets every point, G summed by an all-reduce
        h->dist_pairs = true;
        h->Nc = P.npts;
        h->e0 = 0;
        h->e1 = P.ncell;
      }
    }
  }
  {   // band solver maps (NEXT-2)
    h->d_ent_ptr.assign(P.ngrids, nullptr);
    h->d_ent_slot.assign(P.ngrids, nullptr);
    h->d_ent_pos.assign(P.ngrids, nullptr);
    for (int g = 0; g < P.ngrids; g++)
      if ((rc = upload(h, &h->d_ent_ptr[g], P.grids[g].ent_ptr)) || (rc = upload(h, &h->d_ent_slot[g], P.grids[g].ent_slot)) ||
          (rc = upload(h, &h->d_ent_pos[g], P.grids[g].ent_pos)))
        return bail(rc);
    std::vector<int32_t> perm_all;
    std::vector<int64_t> perm_off, vec_off;
    int64_t off = 0, aoff = 0;
    for (int a = 0; a < h->S; a++) {
      const int g = h->sgrid[a];
      const GridPlan &G = P.grids[g];
      h->band_desc.push_back(
          {off, aoff, h->d_ent_ptr[g], h->d_ent_pos[g], G.ndof, G.band_p, G.band_p + 1, (int)G.ent_slot.size()});
      off += (int64_t)G.ndof * (2 * G.band_p + 1);
      aoff += (int64_t)G.ent_slot.size();
      for (int r = 0; r < G.ndof; r += 8)   // entries of one group of 8 entering rows (kernels_band.cuh)
        h->band_ent_max = std::max(h->band_ent_max, G.ent_ptr[std::min(r + 8, G.ndof)] - G.ent_ptr[r]);
      perm_off.push_back((int64_t)perm_all.size());
      perm_all.insert(perm_all.end(), G.rcm_perm.begin(), G.rcm_perm.end());
      vec_off.push_back(h->soff[a]);
    }
    h->band_bstride = off;
    h->ent_bstride = aoff;
    if ((rc = upload(h, &h->d_band_desc, h->band_desc)) || (rc = upload(h, &h->d_perm_all, perm_all)) ||
        (rc = upload(h, &h->d_perm_off, perm_off)) || (rc = upload(h, &h->d_vec_off, vec_off)))
      return bail(rc);
  }
  h->d_csr.resize(P.ngrids);
  h->d_coo.resize(P.ngrids);
  h->d_mass_csr.assign(P.ngrids, nullptr);
  h->d_mass_coo.assign(P.ngrids, nullptr);
  h->d_adv_csr.assign(P.ngrids, nullptr);
  h->d_adv_coo.assign(P.ngrids, nullptr);
  h->d_rowptr.assign(P.ngrids, nullptr);
  h->d_col.assign(P.ngrids, nullptr);
  for (int g = 0; g < P.ngrids; g++) {
    std::vector<int32_t> col(P.grids[g].col.begin(), P.grids[g].col.end());
    if ((rc = upload(h, &h->d_rowptr[g], P.grids[g].rowptr)) || (rc = upload(h, &h->d_col[g], col))) return bail(rc);
  }
  for (int g = 0; g < P.ngrids; g++) {
    for (int f = 0; f < 2; f++) {
      const GatherMap &m = f == 0 ? P.csr_map[g] : P.coo_map[g];
      auto &d = f == 0 ? h->d_csr[g] : h->d_coo[g];
      if ((rc = upload(h, &d.ptr, m.ptr)) || (rc = upload(h, &d.idx, m.idx)) || (rc = upload(h, &d.w, m.w))) return bail(rc);
      d.nslots = (int64_t)m.ptr.size() - 1;
    }
  }
  for (int f = 0; f < 2; f++) {   // the grids' gather maps with their species factors (tail_kernel)
    std::vector<GatherDev> gms(P.ngrids);
    for (int g = 0; g < P.ngrids; g++) {
      const auto &m = f == 0 ? h->d_csr[g] : h->d_coo[g];
      GatherDev &gd = gms[g];
      gd = GatherDev{};
      gd.ptr = m.ptr;
      gd.idx = m.idx;
      gd.w = m.w;
      gd.nslots = m.nslots;
      gd.nsp = h->spc.grid_nsp[g];
      for (int q = 0; q < gd.nsp; q++) {
        const int sp = h->spc.grid_sp[g][q];
        gd.out_off[q] = f == 0 ? h->snnz_off[sp] : h->scoo_off[sp];
        gd.fD[q] = h->spc.fD[sp];
        gd.fK[q] = h->spc.fK[sp];
      }
    }
    if ((rc = upload(h, &h->d_gmaps[f], gms))) return bail(rc);
  }
  {   // tail_kernel's phased maps: phases of as many cells as fit the shared memory left beside the
      // sum-factorisation scratch (meshes of up to ~128 cells per grid; larger meshes keep two kernels)
    int optin = 0;
    cudaDeviceGetAttribute(&optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, cuda_device);
    const int S = P.p + 1, nb = P.nb;
    const size_t fixed = P.nb == 25 ? tail_smem_bytes<5>(0, 0) : P.nb == 16 ? tail_smem_bytes<4>(0, 0) : tail_smem_bytes<3>(0, 0);
    // 16 KB for straddling-slot partials, 8 KB for the kernel's static tables (phase tables, species)
    const size_t per_cell = sizeof(double) * 2 * nb * nb, cross_reserve = 24 * 1024, static_smem = 8 * 1024;
    const int cap = optin > (int)(fixed + cross_reserve) ? (int)((optin - fixed - cross_reserve) / per_cell) : 0;
    int64_t max_grid_cells = 0;
    for (int g = 0; g < P.ngrids; g++) max_grid_cells = std::max(max_grid_cells, P.grids[g].ncell);
    (void)S;
    if (cap >= 4 && max_grid_cells <= 8LL * cap) {
      bool ok = true;
      for (int f = 0; f < 2 && ok; f++) {
        PhaseMaps pm;
        if (!build_phase_maps(P, f == 0 ? P.csr_map : P.coo_map, cap, pm).empty()) {
          ok = false;
          break;
        }
        auto &m = h->tmaps[f];
        m.max_cells = pm.max_cells;
        m.max_cross = pm.max_cross;
        m.nphases = (int)pm.slot_ptr.size() - 1;
        if (m.nphases > kTailMaxPhases || (size_t)pm.max_cross >= (1u << 26)) {
          ok = false;
          break;
        }
        if ((rc = upload(h, &m.grid_phase_ptr, pm.grid_phase_ptr)) || (rc = upload(h, &m.cell_ptr, pm.cell_ptr)) ||
            (rc = upload(h, &m.slot_ptr, pm.slot_ptr)) || (rc = upload(h, &m.meta, pm.meta)) ||
            (rc = upload(h, &m.idx4, pm.idx4)) || (rc = upload(h, &m.optr, pm.optr)) ||
            (rc = upload(h, &m.oidx, pm.oidx)) || (rc = upload(h, &m.w4, pm.w4)) || (rc = upload(h, &m.ow, pm.ow)))
          return bail(rc);
        const size_t need = P.nb == 25 ? tail_smem_bytes<5>(m.max_cells, m.max_cross)
                            : P.nb == 16 ? tail_smem_bytes<4>(m.max_cells, m.max_cross)
                                         : tail_smem_bytes<3>(m.max_cells, m.max_cross);
        if (need + static_smem > (size_t)optin) ok = false;
      }
      h->tail_ok = ok;
    }
  }
  switch (P.nb) {
    case 9: rc = build_mass<9>(h); break;
    case 16: rc = build_mass<16>(h); break;
    case 25: rc = build_mass<25>(h); break;
  }
  if (rc) return bail(rc);
  if (mode == LANDAU_DIST_ELEMENTS) {
    if (!dist->nccl_unique_id) return bail(fail(h, LANDAU_EINVAL, "nccl_unique_id required for element split"));
    if (!load_nccl()) return bail(fail(h, LANDAU_ENCCL, "cannot load libnccl.so.2"));
    ncclUniqueId_ id;
    memcpy(&id, dist->nccl_unique_id, 128);
    int nr = g_nccl.CommInitRank(&h->comm, world, id, rank);
    if (nr != 0) return bail(fail(h, LANDAU_ENCCL, std::string("ncclCommInitRank: ") + g_nccl.GetErrorString(nr)));
  }
  *out = h;
  return LANDAU_OK;
}


// ==================================================================================================
// NEXT-4 completed: the 3D Cartesian Landau Jacobian (landau3d_*, include/landau.h)
// ==================================================================================================
struct landau3d_s {
  int device = 0;
  cudaStream_t stream = nullptr;
  landau::Plan3D P;
  int S = 0;
  landau::Species3D sp{};
  landau::GatherDev gm{};
  double *d_L1 = nullptr, *d_D1 = nullptr, *d_xyz = nullptr, *d_w = nullptr, *d_wTD = nullptr, *d_wTK = nullptr,
         *d_G = nullptr, *d_C = nullptr, *d_mw = nullptr;
  int32_t *d_dofs = nullptr, *d_idx = nullptr;
  int64_t *d_ptr = nullptr;
  float stage_ms[4] = {0, 0, 0, 0};   // field, inner, element, assemble of the last timed build
  bool timing = false;
};

namespace {
void free3d(landau3d_t h) {
  for (void *p : {(void *)h->d_L1, (void *)h->d_D1, (void *)h->d_xyz, (void *)h->d_w, (void *)h->d_wTD, (void *)h->d_wTK,
                  (void *)h->d_G, (void *)h->d_C, (void *)h->d_mw, (void *)h->d_dofs, (void *)h->d_idx, (void *)h->d_ptr})
    if (p) cudaFree(p);
}
template <class T>
int up3d(landau3d_t h, T **dst, const std::vector<T> &src) {
  if (cudaMalloc((void **)dst, std::max<size_t>(src.size(), 1) * sizeof(T)) != cudaSuccess) return LANDAU_ENOMEM;
  if (!src.empty() && cudaMemcpyAsync(*dst, src.data(), src.size() * sizeof(T), cudaMemcpyHostToDevice, h->stream) != cudaSuccess)
    return LANDAU_ECUDA;
  return LANDAU_OK;
}
template <class F>
int guarded3d(landau3d_t h, F &&body) {
  try {
    int prev = -1, cur = 0;
    if (h && cudaGetDevice(&cur) == cudaSuccess && cur != h->device && cudaSetDevice(h->device) == cudaSuccess) prev = cur;
    const int rc = body();
    if (prev >= 0) cudaSetDevice(prev);
    return rc;
  } catch (const std::bad_alloc &) {
    return LANDAU_ENOMEM;
  } catch (...) {
    return LANDAU_EINVAL;
  }
}
template <int S1>
int build3d(landau3d_t h, const double *f, double *J) {
  using namespace landau;
  const Plan3D &P = h->P;
  cudaEvent_t ev[5];
  if (h->timing)
    for (auto &e : ev) cudaEventCreate(&e);
  auto mark = [&](int i) {
    if (h->timing) cudaEventRecord(ev[i], h->stream);
  };
  mark(0);
  const unsigned gf = (unsigned)std::min<int64_t>((P.npts + 127) / 128, 148LL * 16);
  field3d_kernel<S1><<<gf, 128, 0, h->stream>>>(P.npts, f, P.ndof, h->d_dofs, h->d_L1, h->d_D1, 2.0 / P.h, h->d_w, h->sp,
                                                h->d_wTD, h->d_wTK);
  if (cudaGetLastError() != cudaSuccess) return LANDAU_ECUDA;
  mark(1);
  int rc = landau3d_inner(P.npts, h->d_xyz, h->d_wTD, h->d_wTK, h->d_G, h->stream);
  if (rc) return rc;
  mark(2);
  const int64_t ncube = (int64_t)P.ncell * P.ncell * P.ncell;
  element3d_kernel<S1><<<(unsigned)std::min<int64_t>(ncube, 148LL * 8), k3dElThreads, 0, h->stream>>>(
      ncube, h->d_G, P.npts, h->d_w, h->d_L1, h->d_D1, 2.0 / P.h, reinterpret_cast<double2 *>(h->d_C));
  if (cudaGetLastError() != cudaSuccess) return LANDAU_ECUDA;
  mark(3);
  assemble_kernel<S1 * S1 * S1, 1><<<dim3((unsigned)((P.nnz + 127) / 128), 1), 128, 0, h->stream>>>(h->gm, h->d_C, 0, J,
                                                                                                    0, 1);
  if (cudaGetLastError() != cudaSuccess) return LANDAU_ECUDA;
  mark(4);
  if (h->timing) {
    cudaEventSynchronize(ev[4]);
    for (int i = 0; i < 4; i++) cudaEventElapsedTime(&h->stage_ms[i], ev[i], ev[i + 1]);
    for (auto &e : ev) cudaEventDestroy(e);
  }
  return LANDAU_OK;
}
}  // namespace

extern "C" {

int landau3d_create(landau3d_t *out, int32_t ncell, int32_t order, double R, int32_t nspecies, const double *mass,
                    const double *charge, double nu, int32_t cuda_device, void *cuda_stream) {
  if (!out) return LANDAU_EINVAL;
  *out = nullptr;
  if (nspecies < 1 || nspecies > landau::kMaxSpecies || !mass || !charge) return LANDAU_EINVAL;
  for (int a = 0; a < nspecies; a++)
    if (!(mass[a] > 0.0)) return LANDAU_EINVAL;
  landau3d_t h = nullptr;
  int prev = -1;
  const int rc = [&]() -> int {
    try {
      h = new landau3d_s();
      const std::string err = landau::build_plan3d(ncell, order, R, h->P);
      if (!err.empty()) return LANDAU_EINVAL;
      int cur = 0;
      if (cudaGetDevice(&cur) != cudaSuccess) return LANDAU_ECUDA;
      if (cur != cuda_device) {
        if (cudaSetDevice(cuda_device) != cudaSuccess) return LANDAU_ECUDA;
        prev = cur;
      }
      h->device = cuda_device;
      h->stream = (cudaStream_t)cuda_stream;
      h->S = nspecies;
      h->sp.S = nspecies;
      h->gm.nsp = nspecies;
      h->gm.nslots = h->P.nnz;
      for (int a = 0; a < nspecies; a++) {   // a-1 sums and a-3 factors
        const double e2 = charge[a] * charge[a], im = 1.0 / mass[a];
        h->sp.e2[a] = e2;
        h->sp.e2m[a] = e2 * im;
        h->gm.out_off[a] = (int64_t)a * h->P.nnz;
        h->gm.fD[a] = -nu * e2 * im * im;
        h->gm.fK[a] = nu * e2 * im;
      }
      const landau::Plan3D &P = h->P;
      const int64_t ncube = (int64_t)P.ncell * P.ncell * P.ncell;
      int r;
      if ((r = up3d(h, &h->d_L1, P.L1)) || (r = up3d(h, &h->d_D1, P.D1)) || (r = up3d(h, &h->d_xyz, P.xyz)) ||
          (r = up3d(h, &h->d_w, P.w)) || (r = up3d(h, &h->d_dofs, P.dofs)) || (r = up3d(h, &h->d_ptr, P.map.ptr)) ||
          (r = up3d(h, &h->d_idx, P.map.idx)) || (r = up3d(h, &h->d_mw, P.map.w)))
        return r;
      if (cudaMalloc(&h->d_wTD, sizeof(double) * P.npts) != cudaSuccess ||
          cudaMalloc(&h->d_wTK, sizeof(double) * 3 * P.npts) != cudaSuccess ||
          cudaMalloc(&h->d_G, sizeof(double) * 9 * P.npts) != cudaSuccess ||
          cudaMalloc(&h->d_C, sizeof(double) * 2 * ncube * P.nb * P.nb) != cudaSuccess)
        return LANDAU_ENOMEM;
      h->gm.ptr = h->d_ptr;
      h->gm.idx = h->d_idx;
      h->gm.w = h->d_mw;
      if (cudaStreamSynchronize(h->stream) != cudaSuccess) return LANDAU_ECUDA;
      return LANDAU_OK;
    } catch (const std::bad_alloc &) {
      return LANDAU_ENOMEM;
    } catch (...) {
      return LANDAU_EINVAL;
    }
  }();
  if (rc != LANDAU_OK) {
    if (h) {
      free3d(h);
      delete h;
    }
  } else {
    *out = h;
  }
  if (prev >= 0) cudaSetDevice(prev);
  return rc;
}

int landau3d_get_sizes(landau3d_t h, int64_t *ndof, int64_t *npoints, int64_t *nnz) {
  if (!h) return LANDAU_EINVAL;
  if (ndof) *ndof = h->P.ndof;
  if (npoints) *npoints = h->P.npts;
  if (nnz) *nnz = h->P.nnz;
  return LANDAU_OK;
}

int landau3d_get_pattern(landau3d_t h, int64_t *rowptr, int32_t *col) {
  if (!h) return LANDAU_EINVAL;
  if (rowptr) std::copy(h->P.rowptr.begin(), h->P.rowptr.end(), rowptr);
  if (col) std::copy(h->P.col.begin(), h->P.col.end(), col);
  return LANDAU_OK;
}

int landau3d_get_nodes(landau3d_t h, double *xyz) {
  if (!h || !xyz) return LANDAU_EINVAL;
  const landau::Plan3D &P = h->P;
  const int64_t M = (int64_t)P.ncell * P.p + 1, nd = P.ndof;
  const double d = P.h / P.p;
  for (int64_t iz = 0; iz < M; iz++)
    for (int64_t iy = 0; iy < M; iy++)
      for (int64_t ix = 0; ix < M; ix++) {
        const int64_t k = (iz * M + iy) * M + ix;
        xyz[k] = -P.R + ix * d;
        xyz[nd + k] = -P.R + iy * d;
        xyz[2 * nd + k] = -P.R + iz * d;
      }
  return LANDAU_OK;
}

int landau3d_jacobian(landau3d_t h, const double *f_dev, double *J_dev) {
  if (!h || !f_dev || !J_dev) return LANDAU_EINVAL;
  return guarded3d(h, [&]() -> int { return h->P.s1 == 3 ? build3d<3>(h, f_dev, J_dev) : build3d<4>(h, f_dev, J_dev); });
}

int landau3d_set_timing(landau3d_t h, int32_t enable) {
  if (!h) return LANDAU_EINVAL;
  h->timing = enable != 0;
  return LANDAU_OK;
}

int landau3d_get_timing(landau3d_t h, float *ms4) {
  if (!h || !ms4) return LANDAU_EINVAL;
  for (int i = 0; i < 4; i++) ms4[i] = h->stage_ms[i];
  return LANDAU_OK;
}

void landau3d_destroy(landau3d_t h) {
  if (!h) return;
  try {
    cudaSetDevice(h->device);
    if (h->stream) cudaStreamSynchronize(h->stream);
    free3d(h);
    delete h;
  } catch (...) {
  }
}

}  // extern "C"
