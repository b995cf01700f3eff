// seis.cu — runtime + C ABI (include/seis.h) of the B200-native hot path.
//
// Product path only: no oracle code, no CPU fallback.  The runtime owns the
// device memory plan (padded z-slab fields, per-point coefficients, compact
// C-PML slabs, the HBM snapshot pool), drives Algorithm 1 on the
// caller's stream, and exchanges the 4 ghost planes between z-slabs:
// cudaMemcpyAsync between slabs of one process, NCCL send/recv between ranks.
#include <cuda.h>
#include <cudaTypedefs.h>
#include <cuda_runtime.h>
#include <nccl.h>

#include <algorithm>
#include <cmath>
#include <cstdarg>
#include <cstdio>
#include <cstring>
#include <functional>
#include <map>
#include <string>
#include <vector>

#include "../../include/seis.h"
#include "common.cuh"
#include "kernels_acoustic.cuh"
#include "kernels_acoustic_step.cuh"
#include "kernels_aux.cuh"
#include "kernels_elastic.cuh"
#include "kernels_iso.cuh"
#include "kernels_iso2.cuh"

using namespace seis;

// ------------------------------------------------------------------ errors
static thread_local std::string g_err;
static thread_local long long g_launches = 0;
#if SEIS_AS_TRACE
static unsigned long long* g_trace = nullptr;  // SEIS_AS_TRACE builds: fused-step event buffer
static size_t g_trace_n = 0;
#endif

static seis_status fail(seis_status st, const char* fmt, ...) {
  char buf[1024];
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(buf, sizeof buf, fmt, ap);
  va_end(ap);
  g_err = buf;
  return st;
}

#define CK(call)                                                                          \
  do {                                                                                    \
    cudaError_t e_ = (call);                                                              \
    if (e_ != cudaSuccess)                                                                \
      return fail(e_ == cudaErrorMemoryAllocation ? SEIS_ENOMEM : SEIS_ECUDA, "%s: %s (%s:%d)", \
                  #call, cudaGetErrorString(e_), __FILE__, __LINE__);                     \
  } while (0)
#define CKL()                                                                             \
  do {                                                                                    \
    ++g_launches;                                                                         \
    cudaError_t e_ = cudaGetLastError();                                                  \
    if (e_ != cudaSuccess)                                                                \
      return fail(SEIS_ECUDA, "kernel launch: %s (%s:%d)", cudaGetErrorString(e_), __FILE__, \
                  __LINE__);                                                              \
  } while (0)
#define NK(call)                                                                          \
  do {                                                                                    \
    ncclResult_t r_ = (call);                                                             \
    if (r_ != ncclSuccess)                                                                \
      return fail(SEIS_ENCCL, "%s: %s (%s:%d)", #call, ncclGetErrorString(r_), __FILE__, __LINE__); \
  } while (0)
#define TRY(expr)                      \
  do {                                 \
    seis_status s_ = (expr);           \
    if (s_ != SEIS_OK) return s_;      \
  } while (0)

// ------------------------------------------------------------ profiling
// Per-kernel CUDA-event timing (seis_profile / seis_profile_read): an event pair
// recorded on the launching stream around every launch of a stencil / aux kernel (eager
// launches), or -- graph-sampled mode, seis_profile(S > 1) -- around the launches of every
// S-th time step of a forward shot, as event-record nodes INSIDE the shot's CUDA graph, read
// back after every replay (the timed path stays the production graph).
namespace prof {
constexpr int NK = 11;
static bool on = false;
static int sample = 1;          // 1: every launch, eager; S > 1: graph-sampled every S-th step
static bool sample_now = true;  // (graph-sampled) this time step is bracketed
static int epoch = 0;           // seis_profile resets: part of the graph key (the events are reused)
static std::vector<cudaEvent_t> ev[NK];  // start, stop, start, stop, ...
static size_t used[NK] = {};
static size_t glo[NK] = {}, ghi[NK] = {};  // (graph-sampled) pairs of the current graph
static double acc_ms[NK] = {};
static long long acc_n[NK] = {};
static cudaEvent_t get(int k) {
  if (used[k] == ev[k].size()) {
    cudaEvent_t e;
    cudaEventCreate(&e);
    ev[k].push_back(e);
  }
  return ev[k][used[k]++];
}
struct Scope {
  int k;
  cudaStream_t st;
  bool rec;
  // (under stream capture, the External flag makes the record an event-record NODE of the
  // graph, replayed with it, instead of a capture-internal dependency marker; outside a
  // capture the flag is not allowed)
  static void record(cudaEvent_t e, cudaStream_t s) {
    cudaStreamCaptureStatus cs = cudaStreamCaptureStatusNone;
    cudaStreamIsCapturing(s, &cs);
    cudaEventRecordWithFlags(e, s, cs == cudaStreamCaptureStatusActive ? cudaEventRecordExternal : cudaEventRecordDefault);
  }
  Scope(int k_, cudaStream_t s) : k(k_), st(s), rec(on && sample_now) {
    if (rec) record(get(k), st);
  }
  ~Scope() {
    if (rec) record(get(k), st);
  }
};
// (graph-sampled) add the pairs of the replay that just completed
static cudaError_t harvest() {
  for (int k = 0; k < NK; ++k)
    for (size_t p = glo[k]; p + 1 < ghi[k]; p += 2) {
      float ms = 0.f;
      cudaError_t e = cudaEventElapsedTime(&ms, ev[k][p], ev[k][p + 1]);
      if (e != cudaSuccess) return e;
      acc_ms[k] += ms;
      ++acc_n[k];
    }
  return cudaSuccess;
}
}  // namespace prof
#define PROF(id, st) prof::Scope prof_scope_(id, st)

// ------------------------------------------------------------------ types
struct seis_comm {
  ncclComm_t nccl = nullptr;  // nullptr: peer-only communicator (seis_comm_create_peer)
  int nranks = 1, rank = 0, device = 0;
  double vmax = 0.0;          // peer-only: the caller's global max vp (NCCL reduces it itself)
};

namespace {

// Tile rows per kernel (tools/sweep.py measures the alternatives on a B200).
#ifndef SEIS_BYI
#define SEIS_BYI 8
#endif
#ifndef SEIS_BYV
#define SEIS_BYV 16  // (r02 sweep: ac_v 0.756 vs 0.762 ms at C2 with 8 rows, profiles/r02_sweep_byv.jsonl)
#endif
#ifndef SEIS_BYP
#define SEIS_BYP 8
#endif
#ifndef SEIS_BYE
#define SEIS_BYE (SEIS_EL_WS ? 15 : 8)
#endif
constexpr int BYI = SEIS_BYI;  // ISO step (block 16 x BYI threads, 4 x-points each)
constexpr int BYV = SEIS_BYV;  // acoustic V (block 16 x BYV)
constexpr int BYP = SEIS_BYP;  // acoustic P (block 16 x BYP)
constexpr int BYE = SEIS_BYE;
constexpr int NPSI = 18;

struct Slab {
  Dims d{};
  std::vector<float*> fld;   // padded state fields
  float* m = nullptr;        // ISO
  float* kdt = nullptr;      // ACOUSTIC dt K / h
  float* rho = nullptr;      // ACOUSTIC density (z ghosts filled from the neighbour slabs)
  float *l2m = nullptr, *wmu = nullptr;  // ELASTIC: dt (lam + 2 mu) / h and h / (dt mu)
  float* psi[NPSI] = {};
  // TMA descriptors of every operand tile the kernels stage:
  // "t" = tile with x/y halo, "c" = interior (centre) tile 32 x BY
  CUtensorMap iso_ut[2], iso_uc[2], iso_m;                              // ISO
  CUtensorMap i2_t[2], i2_c[2], i2_m;  // ISO 2-step kernel: u tiles (+ halo 4), u / m interior
  CUtensorMap ac_pt, ac_qc[3], ac_rt, ac_rc, ac_pc;        // ACOUSTIC V
  CUtensorMap ac_qxt, ac_qyt, ac_ppc, ac_qzc, ac_kc;        // ACOUSTIC P
  CUtensorMap el_sxxt, el_sxyt, el_sxzt, el_syyt, el_syzt, el_vc[3], el_rt, el_rc;  // ELASTIC V
  CUtensorMap el_vt[3], el_sc[6], el_l2m, el_w;                           // ELASTIC S
  CUtensorMap as_pt, as_q[3], as_rt, as_rz, as_pq, as_qxn, as_qyn, as_k;  // ACOUSTIC fused step
  int cur = 0;               // ISO: fld[cur] = u^n
  int zc = 1, nzch = 1;      // z-chunking of the stencil launches
  // shot tables
  long long src_o = -1;
  float src_scale = 0.f;
  int nrec_own = 0;
  long long* d_rec_off = nullptr;
  int* d_rec_id = nullptr;
  // backward-phase injection groups (distinct receiver nodes, CSR members), split by the
  // z-chunk that owns the node: [0] = first / last chunk (injected before the overlapped
  // ghost exchange), [1] = interior chunks
  struct Groups {
    int n = 0;
    long long* off = nullptr;
    float* scale = nullptr;
    int* start = nullptr;
    int* mem = nullptr;
    int* surf = nullptr;     // ELASTIC: group node on the free surface
    int* sidx = nullptr;     // ISO O6b: split-storage index of the node (-1 outside the layers)
  } grp[2];
  float* snap = nullptr;     // nsnap * nzl*ny*nx (points into the model's pool)
  Ghost gh[9];               // direct ghost-plane stores per field index (f4)
  // ISO split-field PML (O6b): 6 x spn floats, see IsoArgs::sp
  float* sp = nullptr;
  long long spn = 0;
  int spx = 0, spy = 0;      // x-slab / y-slab region sizes (offsets of the y / z regions)
};

template <class T>
cudaError_t dmalloc(T** p, size_t n) {
  return cudaMalloc((void**)p, std::max<size_t>(n, 1) * sizeof(T));
}

}  // namespace

struct seis_model {
  seis_grid g{};
  seis_kind kind = SEIS_ISO;
  int device = 0;
  seis_comm* comm = nullptr;
  int rank = 0, nranks = 1;
  int pz0 = 0, pnzl = 0;       // this process's z-range
  double vmax = 0.0;           // global max vp
  std::vector<Slab> slabs;
  std::vector<void*> allocs;   // every cudaMalloc of the model
  // 1D coefficient arrays (global index)
  float *edx = nullptr, *edy = nullptr, *edz = nullptr;      // ISO eta*dt
  float* spco[3] = {};        // ISO O6b per-axis update coefficients [3][NP] (A, B, C), see IsoArgs
  int spnp[3] = {};           // their padded lengths NP
  CpmlAxis cp[3] = {};                                       // C-PML
  int W = 0;                   // C-PML slab width per face
  // host copies of this process's model slab (point scales for sources/receivers)
  std::vector<float> hvp, hvs, hrho;
  std::vector<double> eta1[3];  // ISO eta per axis (double, host)
  // snapshot pool
  float* pool = nullptr;
  size_t pool_elems = 0;
  // staging buffers
  float* stage = nullptr;
  size_t stage_elems = 0;
  void* rxb = nullptr;      // resident small-grid ISO path: per-brick halo exchange buffers
  size_t rxb_n = 0;         // (bytes)
  unsigned rxb_base = 0;    // tag base (monotonic over shots: each shot uses base + 1 .. base + nt)
  const float* hwav = nullptr;  // host wavelet of the current call
  float* dwav = nullptr;        // its device copy (uploaded by every call, read by the source add)
  size_t dwav_n = 0;
  int last_nt = 0;
  // shot-table cache and the CUDA graph of the last forward_model.  The gather tables
  // (d_rec_off / d_rec_id, captured by the graph) and the backward-injection groups have
  // separate keys: a migrate between two forward_model calls rebuilds only the groups, and any
  // rebuild of the gather tables destroys the graph that holds their pointers.
  uint64_t fwd_key = 0, bwd_key = 0;
  uint64_t shot_key = 0;              // fwd_key of the current call (part of the graph key)
  std::vector<int> gcur;              // S.cur of every slab after the captured shot (replay)
  cudaStream_t cap = nullptr;       // capture stream (the legacy stream cannot be captured)
  cudaGraphExec_t gexec = nullptr;
  uint64_t gkey = 0;
  // overlapped ghost exchange: side stream + fork / join events
  cudaStream_t xs = nullptr;
  cudaEvent_t ev_fork = nullptr, ev_join = nullptr;
  // ISO split-field PML: the plain-kernel region runs on its own stream, concurrently with the
  // split-field region (SEIS_SPML_CONC=0: one after the other on the compute stream)
  cudaStream_t sps = nullptr;
  cudaEvent_t ev_spf = nullptr, ev_spj = nullptr;
  bool no_overlap = false;  // SEIS_NO_OVERLAP=1: serial exchange (A/B measurements)
  // ACOUSTIC fused step (f1, kernels_acoustic_step.cuh): one persistent launch per time step,
  // one CTA per 64 x 32 tile, all co-resident; ntx x nty tiles, per-tile progress counters
  bool ac_step = false;
  int as_ntx = 0, as_nty = 0;
  unsigned* as_cnt = nullptr;
  bool iso2 = false;  // f1: ISO forward steps in pairs (kernels_iso2.cuh)
  int i2_ntx = 0, i2_nty = 0;
  unsigned* i2_cnt = nullptr;
  long long g_launches = 0;
  // f4 direct ghost stores: `direct` = the faces between the slabs of this
  // process are written by the producing kernels (no copies); `peer` = the rank faces too,
  // through CUDA IPC mappings of the neighbours' fields, ordered by flag words written and
  // waited on with stream memory operations (no NCCL in the step)
  bool direct = false;
  bool peer = false;
  uint32_t* flags = nullptr;      // [0] written by the rank above, [1] by the rank below
  uint32_t* rflag_lo = nullptr;   // the rank above's flags[1] (mapped)
  uint32_t* rflag_hi = nullptr;   // the rank below's flags[0] (mapped)
  uint32_t sig = 0;               // signals issued so far (same sequence on every rank)
  std::vector<void*> ipc_open;    // mapped neighbour allocations
};

namespace {

// ------------------------------------------------------------ helpers
seis_status alloc_track(seis_model* M, void** p, size_t bytes) {
  cudaError_t e = cudaMalloc(p, std::max<size_t>(bytes, 4));
  if (e != cudaSuccess) {
    cudaGetLastError();
    return fail(SEIS_ENOMEM, "cudaMalloc(%zu bytes): %s", bytes, cudaGetErrorString(e));
  }
  M->allocs.push_back(*p);
  return SEIS_OK;
}

// Padded field: ghosts zero, x = 0 of each row 128-byte aligned.
seis_status alloc_padded(seis_model* M, const Dims& d, float** out, cudaStream_t st) {
  size_t elems = (size_t)d.PS * (size_t)(d.nzl + 2 * GZ);
  void* base = nullptr;
  TRY(alloc_track(M, &base, elems * sizeof(float) + 128));
  CK(cudaMemsetAsync(base, 0, elems * sizeof(float) + 128, st));
  *out = (float*)((char*)base + 112);  // (base + 112 + 4*G) % 128 == 0
  return SEIS_OK;
}

int roundup(int a, int b) { return (a + b - 1) / b * b; }

uint64_t fnv1a(const void* p, size_t n, uint64_t h = 1469598103934665603ULL) {
  const unsigned char* c = static_cast<const unsigned char*>(p);
  for (size_t i = 0; i < n; ++i) h = (h ^ c[i]) * 1099511628211ULL;
  return h;
}

// cuTensorMapEncodeTiled through the runtime's driver entry point (no libcuda link).
PFN_cuTensorMapEncodeTiled_v12000 g_encode = nullptr;

seis_status make_map(CUtensorMap* m, float* base, const Dims& d, int bw, int bh, int bd = 1) {
  if (!g_encode) {
    cudaDriverEntryPointQueryResult q;
    void* fn = nullptr;
    CK(cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fn, cudaEnableDefault, &q));
    if (q != cudaDriverEntryPointSuccess || !fn) return fail(SEIS_ECUDA, "cuTensorMapEncodeTiled unavailable");
    g_encode = (PFN_cuTensorMapEncodeTiled_v12000)fn;
  }
  cuuint64_t dims[3] = {(cuuint64_t)d.PX, (cuuint64_t)d.PY, (cuuint64_t)(d.nzl + 2 * GZ)};
  cuuint64_t str[2] = {(cuuint64_t)d.PX * 4, (cuuint64_t)d.PS * 4};
  cuuint32_t box[3] = {(cuuint32_t)bw, (cuuint32_t)bh, (cuuint32_t)bd};
  cuuint32_t es[3] = {1, 1, 1};
  // L2 sector promotion of the tile loads (SEIS_L2PROMO = 0 none, 1 64 B, 2 128 B, 3 256 B: sweeps)
  static const int promo_env = getenv("SEIS_L2PROMO") ? atoi(getenv("SEIS_L2PROMO")) : -1;
  const CUtensorMapL2promotion promo =
      promo_env == 0 ? CU_TENSOR_MAP_L2_PROMOTION_NONE
      : promo_env == 1 ? CU_TENSOR_MAP_L2_PROMOTION_L2_64B
      : promo_env == 3 ? CU_TENSOR_MAP_L2_PROMOTION_L2_256B
                       : CU_TENSOR_MAP_L2_PROMOTION_L2_128B;
  CUresult r = g_encode(m, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 3, base, dims, str, box, es,
                        CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE, promo,
                        CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) return fail(SEIS_ECUDA, "cuTensorMapEncodeTiled failed (%d)", (int)r);
  return SEIS_OK;
}

Dims make_dims(const seis_grid& g, int z0, int nzl) {
  Dims d;
  d.nx = g.nx;
  d.ny = g.ny;
  d.nzl = nzl;
  d.nz = g.nz;
  d.z0 = z0;
  d.PX = roundup(roundup(g.nx, std::max(TXV, TXE)) + 2 * G, 32);
  d.PY = roundup(g.ny, 32) + 2 * G;  // any tile height up to 32
  d.PS = (long long)d.PX * d.PY;
  return d;
}

bool is_device_ptr(const void* p) {
  cudaPointerAttributes a;
  if (cudaPointerGetAttributes(&a, p) != cudaSuccess) {
    cudaGetLastError();
    return false;
  }
  return a.type == cudaMemoryTypeDevice || a.type == cudaMemoryTypeManaged;
}

// Courant bounds of the 8th-order schemes in 3D (O5):
//   ISO leapfrog: v dt/h <= 2/sqrt(3 * sum|c|),  sum|c| over one axis = |c0| + 2 sum|c_m|
//   staggered:    v dt/h <= 1/(sqrt(3) * sum|d_m|)
double courant_limit(seis_kind k) {
  const double c[5] = {205.0 / 72.0, 8.0 / 5.0, 1.0 / 5.0, 8.0 / 315.0, 1.0 / 560.0};
  const double d[4] = {1225.0 / 1024.0, 245.0 / 3072.0, 49.0 / 5120.0, 5.0 / 7168.0};
  if (k == SEIS_ISO) {
    // max of -symbol at k h = pi per axis: c0 + 2 sum c_m cos(m pi) -> |c0| + 2 sum |c_m| (alternating)
    double s = c[0] + 2.0 * (c[1] + c[2] + c[3] + c[4]);
    return 2.0 / std::sqrt(3.0 * s);
  }
  return 1.0 / (std::sqrt(3.0) * (d[0] + d[1] + d[2] + d[3]));
}

// O6: eta_d(xi) = eta_max xi^2, eta_max = 3 vmax ln(1/R) / (2 nb h), xi = layer depth / nb.
double layer_xi(double x, int N, int nb, bool lo, bool hi) {
  double xi = 0.0;
  if (lo && nb - x > xi) xi = nb - x;
  if (hi && x - (N - 1 - nb) > xi) xi = x - (N - 1 - nb);
  xi /= (double)nb;
  return xi > 1.0 ? 1.0 : xi;
}

// O7 (K&M 2007, kappa = 1): d = d0 xi^2, alpha = pi f (1 - xi), b = exp(-(d+alpha) dt),
// a = d (b - 1)/(d + alpha) (0 where d = 0).
void cpml_coef(double xi, double d0, double f, double dt, float* a, float* b) {
  double dd = d0 * xi * xi;
  double al = M_PI * f * (1.0 - xi);
  double bb = std::exp(-(dd + al) * dt);
  *b = (float)bb;
  *a = (float)(dd > 0.0 ? dd * (bb - 1.0) / (dd + al) : 0.0);
}

seis_status upload_padded_from_host(seis_model* M, const Dims& d, const std::vector<float>& host,
                                    float** out, cudaStream_t st) {
  TRY(alloc_padded(M, d, out, st));
  size_t n = (size_t)d.nzl * d.ny * d.nx;
  float* tmp = nullptr;
  CK(cudaMalloc(&tmp, n * sizeof(float)));
  CK(cudaMemcpyAsync(tmp, host.data(), n * sizeof(float), cudaMemcpyHostToDevice, st));
  pad_kernel<<<1024, 256, 0, st>>>(*out, tmp, d);
  CKL();
  CK(cudaStreamSynchronize(st));
  CK(cudaFree(tmp));
  return SEIS_OK;
}

// Opt every TMA-ring kernel into its dynamic shared-memory footprint (once per process).
seis_status set_smem_attrs() {
  static bool done = false;
  if (done) return SEIS_OK;
#define SMEM_ATTR(fn, bytes) CK(cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)(bytes)))
  SMEM_ATTR((iso_step_kernel<BYI, false, false>), IsoStage<BYI>::smem_bytes());
  SMEM_ATTR((iso_step_kernel<BYI, true, false>), IsoStage<BYI>::smem_bytes());
  SMEM_ATTR((iso_step_kernel<BYI, false, true>), IsoStage<BYI>::smem_bytes());
  SMEM_ATTR((iso_step_kernel<BYI, false, false, true>), IsoStage<BYI>::smem_bytes_spml());
  SMEM_ATTR((iso_step_kernel<BYI, true, false, true>), IsoStage<BYI>::smem_bytes_spml());
  SMEM_ATTR((iso_step_kernel<BYI, false, true, true>), IsoStage<BYI>::smem_bytes_spml());
  SMEM_ATTR((iso_step_kernel<BYI, false, false, false, false>), IsoStage<BYI>::smem_bytes());
  SMEM_ATTR((iso_step_kernel<BYI, true, false, false, false>), IsoStage<BYI>::smem_bytes());
  SMEM_ATTR((iso_step_kernel<BYI, false, true, false, false>), IsoStage<BYI>::smem_bytes());
  SMEM_ATTR((iso_step_kernel<BYI, false, false, true, false>), IsoStage<BYI>::smem_bytes_spml());
  SMEM_ATTR((iso_step_kernel<BYI, true, false, true, false>), IsoStage<BYI>::smem_bytes_spml());
  SMEM_ATTR((iso_step_kernel<BYI, false, true, true, false>), IsoStage<BYI>::smem_bytes_spml());
  SMEM_ATTR((ac_v_kernel<BYV, false>), AcVStage<BYV>::smem_bytes());
  SMEM_ATTR((ac_v_kernel<BYV, true>), AcVStage<BYV>::smem_bytes());
  SMEM_ATTR((ac_p_kernel<BYP, false>), AcPStage<BYP>::smem_bytes());
  SMEM_ATTR((ac_p_kernel<BYP, true>), AcPStage<BYP>::smem_bytes());
  SMEM_ATTR((ac_step_kernel<false, false>), AcSLayout::smem_bytes());
  SMEM_ATTR((ac_step_kernel<true, false>), AcSLayout::smem_bytes());
  SMEM_ATTR((ac_step_kernel<false, true>), AcSLayout::smem_bytes());
  SMEM_ATTR((iso2_kernel<false>), Iso2Layout::smem_bytes());
  SMEM_ATTR((iso2_kernel<true>), Iso2Layout::smem_bytes());
  SMEM_ATTR((el_v_kernel<BYE, false, true>), ElVStage<BYE>::smem_bytes());
  SMEM_ATTR((el_v_kernel<BYE, true, true>), ElVStage<BYE>::smem_bytes());
  SMEM_ATTR((el_s_kernel<BYE, false, true>), ElSStage<BYE>::smem_bytes());
  SMEM_ATTR((el_s_kernel<BYE, true, true>), ElSStage<BYE>::smem_bytes());
  SMEM_ATTR((el_v_kernel<BYE, false, false>), ElVStage<BYE>::smem_bytes());
  SMEM_ATTR((el_v_kernel<BYE, true, false>), ElVStage<BYE>::smem_bytes());
  SMEM_ATTR((el_s_kernel<BYE, false, false>), ElSStage<BYE>::smem_bytes());
  SMEM_ATTR((el_s_kernel<BYE, true, false>), ElSStage<BYE>::smem_bytes());
#undef SMEM_ATTR
  done = true;
  return SEIS_OK;
}

// Elastic code-path choice (elastic kernels): without C-PML layers (W = 0) every
// block runs the instantiation without the memory-variable code (fewer instructions and
// registers, no spills: el_s 0.717 -> 0.672 ms at 384^3).  With layers one launch in which
// each block picks its body (region 3): the lean one where its tile and z-chunk hold no layer
// point, the full one elsewhere -- disjoint points, same arithmetic, bitwise unchanged.
// SEIS_EL_REGION=0: the full body everywhere; =1: two launches split by region (measured
// slower: el_v 0.678 -> 0.701 ms at C3, profiles/r02_el_region.log).
template <class Go>
void el_regions(int& region, int W, Go&& go) {
  const char* e = getenv("SEIS_EL_REGION");  // (read per launch: tests flip it between models)
  region = 0;
  if (W <= 0) {
    go(std::false_type{});
  } else if (e && e[0] == '0') {
    go(std::true_type{});
  } else if (e && e[0] == '1') {
    region = 1;
    go(std::false_type{});
    region = 2;
    go(std::true_type{});
    ++g_launches;  // (the caller's CKL counts one)
  } else {
    region = 3;
    go(std::true_type{});
  }
}

// Choose the z-chunk: at most `zt` planes per chunk (short chunks keep the
// blocks resident at any moment on a narrow z-band of the whole plane and shrink the tail of
// the last wave: measured optimum 16 planes for the staggered kernels, 24 for ISO,
// profiles/r01_sweep_zchunk.jsonl), and in any case enough blocks for >= 6 waves of the
// resident slots; chunks of >= 8 planes (the queue warm-up re-reads 8 planes).
// SEIS_ZCHUNK_MAX overrides zt (sweeps).
// zex: planes per face the decomposition exchanges (0 = one slab, no exchange).  The first and
// the last chunk of a slab must then each hold >= zex planes: the overlapped pipeline runs
// them before the exchange (run_phase), and with direct ghost stores they are the only
// kernels that store into a neighbour's ghost planes.
void choose_chunks(Slab& s, int resident_per_sm, int nsm, int tw, int by, int zt, int zex) {
  const long long bxy = (long long)((s.d.nx + tw - 1) / tw) * ((s.d.ny + by - 1) / by);
  const long long slots = (long long)std::max(1, resident_per_sm) * nsm;
  static const int zenv = getenv("SEIS_ZCHUNK_MAX") ? atoi(getenv("SEIS_ZCHUNK_MAX")) : -1;
  const int zmax = zenv >= 0 ? zenv : zt;
  // minimum chunk: 8 planes; a small (L2-resident, launch-bound) grid may go down to
  // SEIS_ZCHUNK_MIN planes to put more blocks on the SMs (the z-queue warm-up re-reads hit L2)
  static const int zmin_env = getenv("SEIS_ZCHUNK_MIN") ? atoi(getenv("SEIS_ZCHUNK_MIN")) : -1;
  // (profiles/r01_c1_sweep.jsonl: C1 64^3 ISO 36.6 -> 58.4 Gpts/s with 2-plane chunks)
  const bool small = (double)s.d.nx * s.d.ny * s.d.nzl < 16.0 * 1024 * 1024;
  const int zmin = std::max(zmin_env > 0 ? zmin_env : (small ? 2 : 8), zex);
  int c = 1;
  while (bxy * c < 6 * slots && (s.d.nzl + c) / (c + 1) >= zmin) ++c;
  if (zmax >= 8)
    while ((s.d.nzl + c - 1) / c > zmax) ++c;
  s.zc = (s.d.nzl + c - 1) / c;
  s.nzch = (s.d.nzl + s.zc - 1) / s.zc;
  if (zex > 0) {
    s.zc = std::max(s.zc, std::min(zex, s.d.nzl));
    s.nzch = (s.d.nzl + s.zc - 1) / s.zc;
    while (s.nzch > 1 && s.d.nzl - (s.nzch - 1) * s.zc < zex) {  // a short last chunk
      ++s.zc;
      s.nzch = (s.d.nzl + s.zc - 1) / s.zc;
    }
  }
}

int nfields(seis_kind k) { return k == SEIS_ISO ? 2 : (k == SEIS_ACOUSTIC ? 4 : 9); }
int npsi_of(seis_kind k) { return k == SEIS_ACOUSTIC ? 6 : (k == SEIS_ELASTIC ? 18 : 0); }
// axis of each C-PML memory array: ACOUSTIC psi_p (x,y,z), psi_q (x,y,z); ELASTIC in the
// oracle's order
int psi_axis(seis_kind k, int t) {
  static const int el_axis[18] = {0, 1, 2, 0, 1, 2, 0, 1, 2, 0, 1, 2, 1, 0, 2, 0, 2, 1};
  return k == SEIS_ACOUSTIC ? t % 3 : el_axis[t];
}

// Ghost-plane exchange between the slabs of this process and, with a
// communicator, with the neighbouring ranks: `np` contiguous planes per face of
// each array `arr(slab)` (a field, or a coefficient array at create time).
using ArrFn = std::function<float*(Slab&)>;

// `state`: the arrays are propagating fields, whose ghost planes the producing kernels store
// directly when M->direct (in-process faces) / M->peer (rank faces) is set (f4); coefficient
// arrays (create time) always travel by copy / NCCL.
seis_status exchange_arrays(seis_model* M, const std::vector<ArrFn>& arrs, int np, cudaStream_t st,
                            bool state = false) {
  const bool local = M->slabs.size() > 1 && !(state && M->direct);
  const bool ranks = M->comm && M->comm->nccl && M->nranks > 1 && !(state && M->peer);
  if (!local && !ranks) return SEIS_OK;
  PROF(7, st);
  for (size_t s = 0; local && s + 1 < M->slabs.size(); ++s) {
    Slab& A = M->slabs[s];
    Slab& B = M->slabs[s + 1];
    const size_t n = (size_t)np * A.d.PS;
    for (const ArrFn& arr : arrs) {
      float* fa = arr(A);
      float* fb = arr(B);
      // A's bottom ghosts (k = nzl .. nzl+np-1) <- B's planes 0 .. np-1
      CK(cudaMemcpyAsync(fa + (size_t)(A.d.nzl + GZ) * A.d.PS, fb + (size_t)GZ * B.d.PS,
                         n * sizeof(float), cudaMemcpyDeviceToDevice, st));
      // B's top ghosts (k = -np .. -1) <- A's planes nzl-np .. nzl-1
      CK(cudaMemcpyAsync(fb + (size_t)(GZ - np) * B.d.PS, fa + (size_t)(A.d.nzl + GZ - np) * A.d.PS,
                         n * sizeof(float), cudaMemcpyDeviceToDevice, st));
    }
  }
  if (ranks) {
    Slab& top = M->slabs.front();
    Slab& bot = M->slabs.back();
    const size_t n = (size_t)np * top.d.PS;
    NK(ncclGroupStart());
    for (const ArrFn& arr : arrs) {
      float* ft = arr(top);
      float* fbm = arr(bot);
      if (M->rank > 0) {
        NK(ncclSend(ft + (size_t)GZ * top.d.PS, n, ncclFloat, M->rank - 1, M->comm->nccl, st));
        NK(ncclRecv(ft + (size_t)(GZ - np) * top.d.PS, n, ncclFloat, M->rank - 1, M->comm->nccl, st));
      }
      if (M->rank < M->nranks - 1) {
        NK(ncclSend(fbm + (size_t)(bot.d.nzl + GZ - np) * bot.d.PS, n, ncclFloat, M->rank + 1,
                    M->comm->nccl, st));
        NK(ncclRecv(fbm + (size_t)(bot.d.nzl + GZ) * bot.d.PS, n, ncclFloat, M->rank + 1,
                    M->comm->nccl, st));
      }
    }
    NK(ncclGroupEnd());
  }
  return SEIS_OK;
}

// np-plane (default 4) exchange of state fields by index
seis_status exchange(seis_model* M, const std::vector<int>& fields, cudaStream_t st, int np = 4) {
  std::vector<ArrFn> arrs;
  for (int f : fields) arrs.push_back([f](Slab& S) { return S.fld[f]; });
  return exchange_arrays(M, arrs, np, st, true);
}

// ---------------------------------------------- f4: rank faces through peer memory
// Stream memory operations (driver entry points, no libcuda link): a signal is a 32-bit
// counter written into the neighbour's flag word after the producing work of a phase; a wait
// blocks the stream until the local flag word reaches the counter (wrap-safe >=).  Every rank
// issues the same sequence of signals, so the counters agree without any exchange.
PFN_cuStreamWriteValue32_v11070 g_wr32 = nullptr;
PFN_cuStreamWaitValue32_v11070 g_wt32 = nullptr;

seis_status memops_init() {
  if (g_wr32 && g_wt32) return SEIS_OK;
  cudaDriverEntryPointQueryResult q;
  void* fn = nullptr;
  CK(cudaGetDriverEntryPoint("cuStreamWriteValue32", &fn, cudaEnableDefault, &q));
  if (q != cudaDriverEntryPointSuccess || !fn) return fail(SEIS_EUNSUPPORTED, "cuStreamWriteValue32 unavailable");
  g_wr32 = (PFN_cuStreamWriteValue32_v11070)fn;
  CK(cudaGetDriverEntryPoint("cuStreamWaitValue32", &fn, cudaEnableDefault, &q));
  if (q != cudaDriverEntryPointSuccess || !fn) return fail(SEIS_EUNSUPPORTED, "cuStreamWaitValue32 unavailable");
  g_wt32 = (PFN_cuStreamWaitValue32_v11070)fn;
  return SEIS_OK;
}

// Tell both neighbours that this rank's work issued on `st` so far (kernels that stored into
// their ghost planes included) is complete: the write is fenced behind the preceding work.
seis_status peer_signal(seis_model* M, cudaStream_t st) {
  if (!M->peer) return SEIS_OK;
  ++M->sig;
  if (M->rflag_lo && g_wr32((CUstream)st, (CUdeviceptr)M->rflag_lo, M->sig, CU_STREAM_WRITE_VALUE_DEFAULT))
    return fail(SEIS_ECUDA, "cuStreamWriteValue32 (rank above) failed");
  if (M->rflag_hi && g_wr32((CUstream)st, (CUdeviceptr)M->rflag_hi, M->sig, CU_STREAM_WRITE_VALUE_DEFAULT))
    return fail(SEIS_ECUDA, "cuStreamWriteValue32 (rank below) failed");
  return SEIS_OK;
}
// Block `st` until both neighbours have issued signal number M->sig.
seis_status peer_wait(seis_model* M, cudaStream_t st) {
  if (!M->peer) return SEIS_OK;
  if (M->rflag_lo && g_wt32((CUstream)st, (CUdeviceptr)(M->flags + 0), M->sig, CU_STREAM_WAIT_VALUE_GEQ))
    return fail(SEIS_ECUDA, "cuStreamWaitValue32 (rank above) failed");
  if (M->rflag_hi && g_wt32((CUstream)st, (CUdeviceptr)(M->flags + 1), M->sig, CU_STREAM_WAIT_VALUE_GEQ))
    return fail(SEIS_ECUDA, "cuStreamWaitValue32 (rank below) failed");
  return SEIS_OK;
}
// Both neighbours have reached the same point of the program: used around every whole-state
// reset / copy (zero, checkpoint save / restore), which must not interleave with the
// neighbours' stores into this rank's ghost planes.
seis_status peer_barrier(seis_model* M, cudaStream_t st) {
  TRY(peer_signal(M, st));
  return peer_wait(M, st);
}

}  // namespace

// ================================================================== C ABI
extern "C" {

const char* seis_version(void) { return "seis-b200 0.1 (sm_100a)"; }

seis_status seis_profile(int32_t enable) {
  const int want = enable > 1 ? enable : 1;
  if (enable) {
    // the same graph-sampled mode again: zero the counters only (the shot graph and its event
    // nodes stay valid, no recapture); anything else: reset the event lists and force new graphs
    const bool same = prof::on && prof::sample > 1 && prof::sample == want;
    for (int k = 0; k < prof::NK; ++k) {
      prof::acc_ms[k] = 0.0;
      prof::acc_n[k] = 0;
      if (!same) prof::used[k] = prof::glo[k] = prof::ghi[k] = 0;
    }
    if (!same) {
      prof::sample = want;
      ++prof::epoch;
    }
  }
  prof::on = enable != 0;
  prof::sample_now = true;
  return SEIS_OK;
}

seis_status seis_profile_read(int32_t kernel, double* total_ms, int64_t* launches) {
  if (kernel < 0 || kernel >= prof::NK || !total_ms || !launches)
    return fail(SEIS_EINVAL, "seis_profile_read: bad arguments");
  if (prof::sample > 1) {  // graph-sampled: accumulated after every replay
    *total_ms = prof::acc_ms[kernel];
    *launches = (int64_t)prof::acc_n[kernel];
    return SEIS_OK;
  }
  double t = 0.0;
  const size_t n = prof::used[kernel] / 2;
  for (size_t p = 0; p < n; ++p) {
    float ms = 0.f;
    CK(cudaEventSynchronize(prof::ev[kernel][2 * p + 1]));
    CK(cudaEventElapsedTime(&ms, prof::ev[kernel][2 * p], prof::ev[kernel][2 * p + 1]));
    t += ms;
  }
  *total_ms = t;
  *launches = (int64_t)n;
  return SEIS_OK;
}
const char* seis_last_error(void) { return g_err.c_str(); }
int64_t seis_last_launch_count(void) { return (int64_t)g_launches; }
#if SEIS_AS_TRACE
// trace builds only (tools/ac_step_trace.py): the fused step's event buffer of the last launch
void* seis_debug_trace(uint64_t* n) {
  cudaDeviceSynchronize();
  *n = g_trace_n;
  return g_trace;
}
#endif

seis_status seis_slab_bounds(int32_t nz, int32_t nranks, int32_t rank, int32_t* z0,
                             int32_t* nz_local) {
  if (!z0 || !nz_local || nranks < 1 || rank < 0 || rank >= nranks || nz < 1)
    return fail(SEIS_EINVAL, "seis_slab_bounds: bad arguments");
  const int base = nz / nranks, rem = nz % nranks;
  *nz_local = base + (rank < rem ? 1 : 0);
  *z0 = rank * base + std::min<int>(rank, rem);
  return SEIS_OK;
}

seis_status seis_comm_unique_id(uint8_t id[128]) {
  if (!id) return fail(SEIS_EINVAL, "null id");
  ncclUniqueId u;
  NK(ncclGetUniqueId(&u));
  std::memcpy(id, u.internal, 128);
  return SEIS_OK;
}

seis_status seis_comm_create(int32_t nranks, int32_t rank, const uint8_t id[128], int32_t device,
                             seis_comm** out) {
  if (!out || !id || nranks < 1 || rank < 0 || rank >= nranks)
    return fail(SEIS_EINVAL, "seis_comm_create: bad arguments");
  CK(cudaSetDevice(device));
  ncclUniqueId u;
  std::memcpy(u.internal, id, 128);
  seis_comm* c = new seis_comm();
  c->nranks = nranks;
  c->rank = rank;
  c->device = device;
  ncclResult_t r = ncclCommInitRank(&c->nccl, nranks, u, rank);
  if (r != ncclSuccess) {
    delete c;
    return fail(SEIS_ENCCL, "ncclCommInitRank: %s", ncclGetErrorString(r));
  }
  *out = c;
  return SEIS_OK;
}

seis_status seis_image_reduce(seis_comm* c, float* image, uint64_t n, void* stream) {
  if (!c || (!image && n)) return fail(SEIS_EINVAL, "seis_image_reduce: null argument");
  if (!c->nccl) return fail(SEIS_EUNSUPPORTED, "seis_image_reduce needs an NCCL communicator (peer-only given)");
  CK(cudaSetDevice(c->device));
  if (!is_device_ptr(image)) return fail(SEIS_EINVAL, "seis_image_reduce: image must be a device buffer");
  cudaStream_t st = (cudaStream_t)stream;
  if (n) NK(ncclAllReduce(image, image, n, ncclFloat, ncclSum, c->nccl, st));
  CK(cudaStreamSynchronize(st));
  return SEIS_OK;
}

seis_status seis_comm_destroy(seis_comm* c) {
  if (!c) return SEIS_OK;
  if (c->nccl) ncclCommDestroy(c->nccl);
  delete c;
  return SEIS_OK;
}

seis_status seis_comm_create_peer(int32_t nranks, int32_t rank, int32_t device, double vmax,
                                  seis_comm** out) {
  if (!out || nranks < 1 || rank < 0 || rank >= nranks || !(vmax > 0.0))
    return fail(SEIS_EINVAL, "seis_comm_create_peer: bad arguments");
  CK(cudaSetDevice(device));
  seis_comm* c = new seis_comm();
  c->nranks = nranks;
  c->rank = rank;
  c->device = device;
  c->vmax = vmax;
  *out = c;
  return SEIS_OK;
}

static seis_status validate_grid(const seis_grid* g, seis_kind kind) {
  if (!g) return fail(SEIS_EINVAL, "null grid");
  if (g->nx < 1 || g->ny < 1 || g->nz < 1) return fail(SEIS_EINVAL, "grid dims must be >= 1");
  if (!(g->h > 0.f) || !(g->dt > 0.f)) return fail(SEIS_EINVAL, "h and dt must be > 0");
  if (g->nb < 0 || 3 * g->nb > std::min(g->nx, std::min(g->ny, g->nz)))
    return fail(SEIS_EINVAL, "nb=%d must satisfy 0 <= 3 nb <= min(nx, ny, nz)", g->nb);
  if (g->nb > 0 && !(g->pml_R > 0.f && g->pml_R < 1.f)) return fail(SEIS_EINVAL, "pml_R in (0,1)");
  if (g->pml_f < 0.f) return fail(SEIS_EINVAL, "pml_f must be >= 0");
  if (kind != SEIS_ISO && kind != SEIS_ACOUSTIC && kind != SEIS_ELASTIC)
    return fail(SEIS_EINVAL, "unknown kind %d", (int)kind);
  if (g->free_surface && kind != SEIS_ELASTIC)
    return fail(SEIS_EUNSUPPORTED, "free_surface is implemented for ELASTIC only");
  if (g->slabs < 1) return fail(SEIS_EINVAL, "slabs must be >= 1");
  if (g->iso_pml != 0 && g->iso_pml != 1) return fail(SEIS_EINVAL, "iso_pml must be 0 or 1");
  if (g->iso_pml && kind != SEIS_ISO) return fail(SEIS_EUNSUPPORTED, "iso_pml applies to ISO only");
  return SEIS_OK;
}

seis_status seis_model_destroy(seis_model* M) {
  if (!M) return SEIS_OK;
  cudaSetDevice(M->device);
  if (M->gexec) cudaGraphExecDestroy(M->gexec);
  if (M->cap) cudaStreamDestroy(M->cap);
  if (M->xs) cudaStreamDestroy(M->xs);
  if (M->sps) cudaStreamDestroy(M->sps);
  if (M->ev_spf) cudaEventDestroy(M->ev_spf);
  if (M->ev_spj) cudaEventDestroy(M->ev_spj);
  if (M->ev_fork) cudaEventDestroy(M->ev_fork);
  if (M->ev_join) cudaEventDestroy(M->ev_join);
  for (void* p : M->ipc_open) cudaIpcCloseMemHandle(p);
  for (Slab& S : M->slabs) {  // shot tables (setup_shot), not in allocs
    cudaFree(S.d_rec_off);
    cudaFree(S.d_rec_id);
    for (auto& G2 : S.grp) {
      cudaFree(G2.off);
      cudaFree(G2.scale);
      cudaFree(G2.start);
      cudaFree(G2.mem);
      cudaFree(G2.surf);
      cudaFree(G2.sidx);
    }
  }
  for (void* p : M->allocs) cudaFree(p);
  delete M;
  return SEIS_OK;
}

static seis_status model_create_impl(seis_model* M, const float* vp, const float* vs,
                                     const float* rho) {
  const seis_grid& g = M->g;
  const seis_kind kind = M->kind;
  cudaStream_t st = 0;
  const size_t plane = (size_t)g.nx * g.ny;
  const size_t npts = plane * M->pnzl;
  // host copies of this process's model slab
  M->hvp.assign(vp, vp + npts);
  if (rho) M->hrho.assign(rho, rho + npts);
  if (vs) M->hvs.assign(vs, vs + npts);
  double vmax = 0.0;
  for (size_t t = 0; t < npts; ++t) {
    if (!(vp[t] > 0.f)) return fail(SEIS_EINVAL, "vp must be > 0 (index %zu)", t);
    vmax = std::max(vmax, (double)vp[t]);
    if (rho && !(rho[t] > 0.f)) return fail(SEIS_EINVAL, "rho must be > 0 (index %zu)", t);
    if (vs && (!(vs[t] >= 0.f) || 2.0 * (double)vs[t] * vs[t] > (double)vp[t] * vp[t]))
      return fail(SEIS_EINVAL, "vs must satisfy 0 <= vs <= vp/sqrt(2) (index %zu)", t);
  }
  // (rho / w at k+1 across rank faces come from the ghost-plane exchange after the upload)
  if (M->comm && M->nranks > 1 && !M->comm->nccl) {
    if (!(M->comm->vmax >= vmax)) return fail(SEIS_EINVAL, "peer communicator vmax %.3f < local max vp %.3f", M->comm->vmax, vmax);
    vmax = M->comm->vmax;
  } else if (M->comm && M->nranks > 1) {
    float* dv = nullptr;
    CK(cudaMalloc(&dv, sizeof(double)));
    CK(cudaMemcpy(dv, &vmax, sizeof(double), cudaMemcpyHostToDevice));
    NK(ncclAllReduce(dv, dv, 1, ncclFloat64, ncclMax, M->comm->nccl, st));
    CK(cudaStreamSynchronize(st));
    CK(cudaMemcpy(&vmax, dv, sizeof(double), cudaMemcpyDeviceToHost));
    CK(cudaFree(dv));
  }
  M->vmax = vmax;
  const double vdt_h = vmax * (double)g.dt / (double)g.h;
  if (vdt_h > courant_limit(kind))
    return fail(SEIS_ECFL, "Courant number vmax dt/h = %.6f exceeds the 8th-order 3D limit %.6f",
                vdt_h, courant_limit(kind));

  const double h = g.h, dt = g.dt;
  const int N3[3] = {g.nx, g.ny, g.nz};
  // 1D absorbing-layer profiles (host, double -> fp32)
  if (kind == SEIS_ISO) {
    float* e1[3];
    for (int ax = 0; ax < 3; ++ax) {
      const int N = N3[ax];
      M->eta1[ax].assign(N, 0.0);
      std::vector<float> hf(N, 0.f);
      if (g.nb > 0) {
        const double emax = 3.0 * vmax * std::log(1.0 / (double)g.pml_R) / (2.0 * g.nb * h);
        for (int i = 0; i < N; ++i) {
          const double xi = layer_xi(i, N, g.nb, true, true);
          M->eta1[ax][i] = emax * xi * xi;
          hf[i] = (float)(M->eta1[ax][i] * dt);
        }
      }
      hf.resize(std::max(N, roundup(N, TXV) + TXV), 0.f);  // float4 loads past nx read zeros
      TRY(alloc_track(M, (void**)&e1[ax], hf.size() * sizeof(float)));
      CK(cudaMemcpy(e1[ax], hf.data(), hf.size() * sizeof(float), cudaMemcpyHostToDevice));
      if (g.iso_pml && g.nb > 0) {
        // O6b: u^(d),n+1 = A u^(d),n - B u^(d),n-1 + C m L_d u^n with e = eta_d dt (as the
        // kernels' fp32 e): A = (2 - e^2)/(1 + e), B = (1 - e)/(1 + e), C = 1/(1 + e), double -> fp32
        const int NP = (int)hf.size();
        std::vector<float> co((size_t)3 * NP, 0.f);
        for (int i = 0; i < NP; ++i) {
          const double e = (double)hf[i];
          co[i] = (float)((2.0 - e * e) / (1.0 + e));
          co[(size_t)NP + i] = (float)((1.0 - e) / (1.0 + e));
          co[(size_t)2 * NP + i] = (float)(1.0 / (1.0 + e));
        }
        TRY(alloc_track(M, (void**)&M->spco[ax], co.size() * sizeof(float)));
        CK(cudaMemcpy(M->spco[ax], co.data(), co.size() * sizeof(float), cudaMemcpyHostToDevice));
        M->spnp[ax] = NP;
      }
    }
    if (g.nb > 0) {
      M->edx = e1[0];
      M->edy = e1[1];
      M->edz = e1[2];
    }
  } else if (g.nb > 0) {
    M->W = g.nb + 1;
    const double d0 = 3.0 * vmax * std::log(1.0 / (double)g.pml_R) / (2.0 * g.nb * h);
    for (int ax = 0; ax < 3; ++ax) {
      const int N = N3[ax];
      const bool lo = !(ax == 2 && g.free_surface);
      std::vector<float> a(N), b(N), ah(N), bh(N);
      for (int i = 0; i < N; ++i) {
        cpml_coef(layer_xi(i, N, g.nb, lo, true), d0, g.pml_f, dt, &a[i], &b[i]);
        cpml_coef(layer_xi(i + 0.5, N, g.nb, lo, true), d0, g.pml_f, dt, &ah[i], &bh[i]);
      }
      float* dv[4];
      const std::vector<float>* hv[4] = {&a, &b, &ah, &bh};
      for (int t = 0; t < 4; ++t) {
        TRY(alloc_track(M, (void**)&dv[t], N * sizeof(float)));
        CK(cudaMemcpy(dv[t], hv[t]->data(), N * sizeof(float), cudaMemcpyHostToDevice));
      }
      M->cp[ax] = CpmlAxis{dv[0], dv[1], dv[2], dv[3]};
    }
  }

  // slabs of this process
  const int ns = g.slabs;
  int dev_sms = 148;
  CK(cudaDeviceGetAttribute(&dev_sms, cudaDevAttrMultiProcessorCount, M->device));
  if (ns > 1 || M->nranks > 1) {
    // every slab must hold the 4 planes its neighbours read as ghosts
    for (int r = 0; r < M->nranks; ++r)
      for (int s = 0; s < ns; ++s) {
        int rz0, rn, lz0, ln;
        seis_slab_bounds(g.nz, M->nranks, r, &rz0, &rn);
        seis_slab_bounds(rn, ns, s, &lz0, &ln);
        if (ln < 4) return fail(SEIS_EINVAL, "z-slab of %d planes: the decomposition needs >= 4", ln);
      }
  }
  M->slabs.resize(ns);
  for (int s = 0; s < ns; ++s) {
    int lz0, lnz;
    seis_slab_bounds(M->pnzl, ns, s, &lz0, &lnz);
    Slab& S = M->slabs[s];
    S.d = make_dims(g, M->pz0 + lz0, lnz);
    const Dims& d = S.d;
    const size_t sp = (size_t)lnz * plane;  // slab points
    const size_t off = (size_t)lz0 * plane;
    S.fld.resize(nfields(kind));
    for (auto& f : S.fld) TRY(alloc_padded(M, d, &f, st));
    // per-point coefficients (double -> fp32), compact then padded on device
    std::vector<float> hc(sp);
    if (kind == SEIS_ISO) {
      for (size_t t = 0; t < sp; ++t) {
        const double v = M->hvp[off + t];
        hc[t] = (float)(v * v * dt * dt / (h * h));
      }
      TRY(upload_padded_from_host(M, d, hc, &S.m, st));
      if (g.iso_pml && g.nb > 0) {  // O6b split components of the layer points
        const long long nbl = g.nb;
        S.spx = (int)((long long)lnz * g.ny * 2 * nbl);
        S.spy = (int)((long long)lnz * 2 * nbl * g.nx);
        S.spn = (long long)S.spx + S.spy + 2 * nbl * g.ny * (long long)g.nx;
        if (S.spn >= 2147483647LL) return fail(SEIS_EUNSUPPORTED, "split-PML storage exceeds 32-bit indexing");
        TRY(alloc_track(M, (void**)&S.sp, (size_t)S.spn * 6 * sizeof(float)));
        CK(cudaMemsetAsync(S.sp, 0, (size_t)S.spn * 6 * sizeof(float), st));
      }
    } else {
      // buoyancy on faces (O8): both V kernels evaluate dt 2/(rho_i + rho_{i+1}) / h on the
      // fly from rho, whose z-ghost planes are exchanged once below
      for (size_t q = 0; q < sp; ++q) hc[q] = M->hrho[off + q];
      TRY(upload_padded_from_host(M, d, hc, &S.rho, st));
      if (kind == SEIS_ACOUSTIC) {
        for (size_t t = 0; t < sp; ++t) {
          const double v = M->hvp[off + t], r = M->hrho[off + t];
          hc[t] = (float)(dt * r * v * v / h);
        }
        TRY(upload_padded_from_host(M, d, hc, &S.kdt, st));
      } else {
        for (size_t t = 0; t < sp; ++t) {
          const double v = M->hvp[off + t], s_ = M->hvs[off + t], r = M->hrho[off + t];
          hc[t] = (float)(dt * r * v * v / h);  // lambda + 2 mu = rho vp^2
        }
        TRY(upload_padded_from_host(M, d, hc, &S.l2m, st));
        // w = h / (dt mu) at nodes (+inf where mu = 0): the S kernel forms the edge mu of O9
        // (harmonic mean of 4 nodes, 0 if any is 0) as 4 / (w0 + w1 + w2 + w3) and
        // dt lam / h = dt (lam + 2 mu) / h - 2 / w; its z-ghost planes are exchanged below
        for (size_t t = 0; t < sp; ++t) {
          const double s_ = M->hvs[off + t], r = M->hrho[off + t], mu = r * s_ * s_;
          hc[t] = mu > 0 ? (float)(h / (dt * mu)) : INFINITY;
        }
        TRY(upload_padded_from_host(M, d, hc, &S.wmu, st));
      }
      // compact C-PML memory slabs (32-bit indices in the kernels)
      if (M->W > 0) {
        const int W = M->W;
        const double big = std::max((double)lnz * g.ny, std::max((double)lnz * g.nx, (double)g.ny * g.nx)) * 2.0 * W;
        if (big >= 2147483647.0) return fail(SEIS_EUNSUPPORTED, "C-PML slab of %.0f points exceeds 32-bit indexing", big);
        const int npsi = npsi_of(kind);
        for (int t = 0; t < npsi; ++t) {
          const int ax = psi_axis(kind, t);
          size_t n;
          if (ax == 0) n = (size_t)lnz * g.ny * 2 * W;
          else if (ax == 1) n = (size_t)lnz * 2 * W * g.nx;
          else n = (size_t)2 * W * g.ny * g.nx;
          TRY(alloc_track(M, (void**)&S.psi[t], n * sizeof(float)));
        }
      }
    }
    // TMA descriptors
    if (kind == SEIS_ISO) {
      for (int t = 0; t < 2; ++t) {
        TRY(make_map(&S.iso_ut[t], S.fld[t], d, TXV + 8, BYI + 8));
        TRY(make_map(&S.iso_uc[t], S.fld[t], d, TXV, BYI));
      }
      TRY(make_map(&S.iso_m, S.m, d, TXV, BYI));
    } else if (kind == SEIS_ACOUSTIC) {
      // V tiles (BYV rows)
      TRY(make_map(&S.ac_pt, S.fld[0], d, TXV + 8, BYV + 8));
      for (int t = 0; t < 3; ++t) TRY(make_map(&S.ac_qc[t], S.fld[1 + t], d, TXV, BYV));
      TRY(make_map(&S.ac_rt, S.rho, d, TXV + 4, BYV + 1));
      TRY(make_map(&S.ac_rc, S.rho, d, TXV, BYV));
      TRY(make_map(&S.ac_pc, S.fld[0], d, TXV, BYV));
      // P tiles (BYP rows)
      TRY(make_map(&S.ac_qxt, S.fld[1], d, TXV + 8, BYP));
      TRY(make_map(&S.ac_qyt, S.fld[2], d, TXV, BYP + 8));
      TRY(make_map(&S.ac_ppc, S.fld[0], d, TXV, BYP));
      TRY(make_map(&S.ac_qzc, S.fld[3], d, TXV, BYP));
      TRY(make_map(&S.ac_kc, S.kdt, d, TXV, BYP));
      // fused step tiles (AS_TX x AS_TY; kernels_acoustic_step.cuh)
      TRY(make_map(&S.as_pt, S.fld[0], d, AS_TX + 8, AS_TY + 8));
      for (int t = 0; t < 3; ++t) TRY(make_map(&S.as_q[t], S.fld[1 + t], d, AS_TX, AS_TY));
      TRY(make_map(&S.as_rt, S.rho, d, AS_TX + 4, AS_TY + 1));
      TRY(make_map(&S.as_rz, S.rho, d, AS_TX, AS_TY));
      TRY(make_map(&S.as_pq, S.fld[0], d, AS_TX, AS_TY));
      TRY(make_map(&S.as_qxn, S.fld[1], d, AS_TX + 8, AS_TY));
      TRY(make_map(&S.as_qyn, S.fld[2], d, AS_TX, AS_TY + 8));
      TRY(make_map(&S.as_k, S.kdt, d, AS_TX, AS_TY));
    } else {
      TRY(make_map(&S.el_sxxt, S.fld[ESXX], d, TXE + 8, BYE));
      TRY(make_map(&S.el_sxyt, S.fld[ESXY], d, TXE + 8, BYE + 8));
      TRY(make_map(&S.el_sxzt, S.fld[ESXZ], d, TXE + 8, BYE));
      TRY(make_map(&S.el_syyt, S.fld[ESYY], d, TXE, BYE + 8));
      TRY(make_map(&S.el_syzt, S.fld[ESYZ], d, TXE, BYE + 8));
      TRY(make_map(&S.el_rt, S.rho, d, TXE + 4, BYE + 1));
      TRY(make_map(&S.el_rc, S.rho, d, TXE, BYE));
      for (int t = 0; t < 3; ++t) {
        TRY(make_map(&S.el_vc[t], S.fld[EVX + t], d, TXE, BYE));
        TRY(make_map(&S.el_vt[t], S.fld[EVX + t], d, TXE + 8, BYE + 8));
      }
      for (int t = 0; t < 6; ++t) TRY(make_map(&S.el_sc[t], S.fld[ESXX + t], d, TXE, BYE));
      TRY(make_map(&S.el_l2m, S.l2m, d, TXE, BYE));
      TRY(make_map(&S.el_w, S.wmu, d, TXE + 4, BYE + 1));
    }
    TRY(set_smem_attrs());
    int occ = 1;
    if (kind == SEIS_ISO)
      cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, iso_step_kernel<BYI, false, false>, NTX * BYI,
                                                    IsoStage<BYI>::smem_bytes());
    else if (kind == SEIS_ACOUSTIC)
      cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, ac_v_kernel<BYV, false>, NTX * BYV,
                                                    AcVStage<BYV>::smem_bytes());
    else
      cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, el_s_kernel<BYE, false, true>, NTX2 * (BYE + EL_WS),
                                                    ElSStage<BYE>::smem_bytes());
    const int zex = (ns > 1 || M->nranks > 1) ? 4 : 0;
    if (kind == SEIS_ELASTIC) choose_chunks(S, occ, dev_sms, TXE, BYE, 16, zex);
    else if (kind == SEIS_ISO) choose_chunks(S, occ, dev_sms, TXV, BYI, 24, zex);
    else choose_chunks(S, occ, dev_sms, TXV, BYV, 16, zex);
  }
  // f1: the fused acoustic step (kernels_acoustic_step.cuh) on a single-slab, single-process
  // model whose tiles can all be resident at once (cooperative launch).  Default: without
  // absorbing layers (nb = 0) and with enough tiles to occupy half the SMs -- there it beats
  // the split pair (512^3: 1.07 vs 1.19 ms per step); with C-PML the layer tiles (about half of
  // them carry memory-variable work) pace the lockstep wavefront and the split pair stays
  // faster.  SEIS_AC_STEP=1 / 0 forces it on (if the tiles fit) / off.  Bitwise
  // the split pair's results either way (tests/test_acoustic_step_gpu.py).
  if (kind == SEIS_ACOUSTIC && ns == 1 && !M->comm) {
    const int ntx = (g.nx + AS_TX - 1) / AS_TX, nty = (g.ny + AS_TY - 1) / AS_TY;
    int occ_s = 0, coop = 0;
    CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ_s, ac_step_kernel<false, false>, AS_THREADS,
                                                     AcSLayout::smem_bytes()));
    CK(cudaDeviceGetAttribute(&coop, cudaDevAttrCooperativeLaunch, M->device));
    const bool fits = coop && occ_s >= 1 && (long long)ntx * nty <= (long long)occ_s * dev_sms;
    const char* e = getenv("SEIS_AC_STEP");
    const bool want = e ? e[0] == '1' : (g.nb == 0 && 2LL * ntx * nty >= dev_sms);
    M->ac_step = fits && want;
    if (M->ac_step) {
      M->as_ntx = ntx;
      M->as_nty = nty;
      void* p = nullptr;
      TRY(alloc_track(M, &p, (size_t)ntx * nty * sizeof(unsigned)));
      M->as_cnt = (unsigned*)p;
    }
  }
  // f1: ISO 2-step temporal blocking (kernels_iso2.cuh) for forward modeling on a single-slab,
  // single-process model without the split-field PML whose tiles are all co-resident
  // (cooperative launch).  Opt-in (SEIS_ISO2=1): bitwise the one-step kernel's results
  // (tests/test_iso2_gpu.py) but slower at 512^3 (0.892 ms per two steps vs 2 x 0.353 ms:
  // 14 warps per SM with two 9-deep register queues are issue / shared-memory-latency bound,
  // DESIGN.md §6 "ISO 2-step").
  if (kind == SEIS_ISO && ns == 1 && !M->comm && !(g.iso_pml && g.nb > 0)) {
    const int ntx = (g.nx + I2_TX - 1) / I2_TX, nty = (g.ny + I2_TY - 1) / I2_TY;
    int occ2 = 0, coop = 0;
    CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ2, iso2_kernel<true>, I2_THREADS,
                                                     Iso2Layout::smem_bytes()));
    CK(cudaDeviceGetAttribute(&coop, cudaDevAttrCooperativeLaunch, M->device));
    const bool fits = coop && occ2 >= 1 && (long long)ntx * nty <= (long long)occ2 * dev_sms;
    const char* e = getenv("SEIS_ISO2");
    M->iso2 = fits && e && e[0] == '1';
    if (M->iso2) {
      Slab& S = M->slabs[0];
      const Dims& d = S.d;
      for (int t = 0; t < 2; ++t) {
        TRY(make_map(&S.i2_t[t], S.fld[t], d, I2_TX + 8, I2_TY + 8));
        TRY(make_map(&S.i2_c[t], S.fld[t], d, I2_TX, I2_TY));
      }
      TRY(make_map(&S.i2_m, S.m, d, I2_TX, I2_TY));
      M->i2_ntx = ntx;
      M->i2_nty = nty;
      void* p = nullptr;
      TRY(alloc_track(M, &p, (size_t)ntx * nty * sizeof(unsigned)));
      M->i2_cnt = (unsigned*)p;
    }
  }
  // f4: the faces between the slabs of this process by direct ghost stores of the producing
  // kernels (SEIS_GHOST_COPY=1 keeps the copy exchange, the A/B alternative).  Not for the
  // fused acoustic step, which exchanges 8 ghost planes of p.
  {
    const char* e = getenv("SEIS_GHOST_COPY");
    M->direct = ns > 1 && !(e && e[0] == '1');
    for (int s = 0; M->direct && s < ns; ++s) {
      Slab& S = M->slabs[s];
      for (size_t f = 0; f < S.fld.size() && f < 9; ++f) {
        if (s > 0) {
          S.gh[f].lo = M->slabs[s - 1].fld[f];
          S.gh[f].loo = (long long)M->slabs[s - 1].d.nzl * S.d.PS;
        }
        if (s + 1 < ns) {
          S.gh[f].hi = M->slabs[s + 1].fld[f];
          S.gh[f].hio = -(long long)S.d.nzl * S.d.PS;
        }
      }
    }
  }
  if (ns > 1 || M->nranks > 1) {
    const char* e = getenv("SEIS_NO_OVERLAP");
    M->no_overlap = e && e[0] == '1';
    CK(cudaStreamCreateWithFlags(&M->xs, cudaStreamNonBlocking));
    CK(cudaEventCreateWithFlags(&M->ev_fork, cudaEventDisableTiming));
    CK(cudaEventCreateWithFlags(&M->ev_join, cudaEventDisableTiming));
  }
  if (kind == SEIS_ACOUSTIC)  // rho(k+1) across slab faces
    TRY(exchange_arrays(M, {[](Slab& S) { return S.rho; }}, 4, st));
  if (kind == SEIS_ELASTIC)  // rho(k+1), w(k+1) across slab faces
    TRY(exchange_arrays(M, {[](Slab& S) { return S.rho; }, [](Slab& S) { return S.wmu; }}, 4, st));
  CK(cudaStreamSynchronize(st));
  return SEIS_OK;
}

seis_status seis_model_create(const seis_grid* grid, seis_kind kind, const float* vp,
                              const float* vs, const float* rho, seis_comm* comm, int32_t device,
                              seis_model** out) {
  if (!out) return fail(SEIS_EINVAL, "null out");
  *out = nullptr;
  TRY(validate_grid(grid, kind));
  if (!vp) return fail(SEIS_EINVAL, "vp is required");
  if ((kind == SEIS_ACOUSTIC || kind == SEIS_ELASTIC) && !rho)
    return fail(SEIS_EINVAL, "rho is required for ACOUSTIC and ELASTIC");
  if (kind == SEIS_ELASTIC && !vs) return fail(SEIS_EINVAL, "vs is required for ELASTIC");
  if (comm && grid->slabs != 1)
    return fail(SEIS_EUNSUPPORTED, "slabs > 1 is the single-process decomposition mode");
  int ndev = 0;
  cudaError_t e = cudaGetDeviceCount(&ndev);
  if (e != cudaSuccess || ndev == 0) {
    cudaGetLastError();
    return fail(SEIS_ECUDA, "no CUDA device: %s", cudaGetErrorString(e));
  }
  if (device < 0 || device >= ndev) return fail(SEIS_EINVAL, "device %d out of range", device);
  CK(cudaSetDevice(device));
  seis_model* M = new seis_model();
  M->g = *grid;
  M->kind = kind;
  M->device = device;
  M->comm = comm;
  M->nranks = comm ? comm->nranks : 1;
  M->rank = comm ? comm->rank : 0;
  int32_t z0, nzl;
  seis_slab_bounds(grid->nz, M->nranks, M->rank, &z0, &nzl);
  M->pz0 = z0;
  M->pnzl = nzl;
  seis_status s = model_create_impl(M, vp, kind == SEIS_ELASTIC ? vs : nullptr,
                                    kind == SEIS_ISO ? nullptr : rho);
  if (s != SEIS_OK) {
    std::string keep = g_err;
    seis_model_destroy(M);
    g_err = keep;
    return s;
  }
  *out = M;
  return SEIS_OK;
}

}  // extern "C"

namespace {
// What a rank publishes for its neighbours' direct ghost stores (f4): CUDA IPC handles of the
// allocation bases of its state fields (field = base + 112 bytes, alloc_padded), of the
// coefficient arrays whose ghost planes the neighbours fill once, and of its flag words.
struct PeerBlob {
  uint32_t magic;
  int32_t kind, rank, nranks, nzl, nfld, PX, PY;
  cudaIpcMemHandle_t fld[9];
  cudaIpcMemHandle_t coef[2];  // rho, w (ELASTIC) -- ACOUSTIC: rho only
  cudaIpcMemHandle_t flags;
};
constexpr uint32_t PEER_MAGIC = 0x50494553u;  // "SEIP"
constexpr size_t PADB = 112;                   // alloc_padded: field = base + 112 bytes

int ncoef(seis_kind k) { return k == SEIS_ISO ? 0 : (k == SEIS_ACOUSTIC ? 1 : 2); }
float* coef_of(Slab& S, int t) { return t == 0 ? S.rho : S.wmu; }

seis_status peer_open(seis_model* M, const cudaIpcMemHandle_t& h, char** p) {
  void* q = nullptr;
  cudaError_t e = cudaIpcOpenMemHandle(&q, h, cudaIpcMemLazyEnablePeerAccess);
  if (e != cudaSuccess) {
    cudaGetLastError();
    return fail(SEIS_ECUDA, "cudaIpcOpenMemHandle: %s", cudaGetErrorString(e));
  }
  M->ipc_open.push_back(q);
  *p = (char*)q;
  return SEIS_OK;
}

seis_status check_blob(const seis_model* M, const uint8_t* b, uint64_t len, int want_rank) {
  if (!b || len < sizeof(PeerBlob)) return fail(SEIS_EINVAL, "peer blob of rank %d missing or short", want_rank);
  PeerBlob p;
  std::memcpy(&p, b, sizeof p);
  const Slab& S = M->slabs.front();
  if (p.magic != PEER_MAGIC || p.kind != (int)M->kind || p.rank != want_rank || p.nranks != M->nranks ||
      p.nfld != (int)S.fld.size() || p.PX != S.d.PX || p.PY != S.d.PY)
    return fail(SEIS_EINVAL, "peer blob does not belong to rank %d of this decomposition", want_rank);
  return SEIS_OK;
}
}  // namespace

extern "C" {

seis_status seis_model_peer_export(seis_model* M, uint8_t* blob, uint64_t cap, uint64_t* len) {
  if (!M || !len) return fail(SEIS_EINVAL, "null argument");
  *len = sizeof(PeerBlob);
  if (!blob) return SEIS_OK;  // size query
  if (cap < sizeof(PeerBlob)) return fail(SEIS_EINVAL, "blob capacity %llu < %zu", (unsigned long long)cap, sizeof(PeerBlob));
  if (!M->comm || M->nranks < 2 || M->slabs.size() != 1)
    return fail(SEIS_EINVAL, "peer halo needs a multi-rank model (one slab per rank)");
  CK(cudaSetDevice(M->device));
  if (!M->flags) {
    void* f = nullptr;
    TRY(alloc_track(M, &f, 256));
    CK(cudaMemset(f, 0, 256));
    M->flags = (uint32_t*)f;
  }
  Slab& S = M->slabs.front();
  PeerBlob p{};
  p.magic = PEER_MAGIC;
  p.kind = (int)M->kind;
  p.rank = M->rank;
  p.nranks = M->nranks;
  p.nzl = S.d.nzl;
  p.nfld = (int)S.fld.size();
  p.PX = S.d.PX;
  p.PY = S.d.PY;
  for (size_t f = 0; f < S.fld.size(); ++f) CK(cudaIpcGetMemHandle(&p.fld[f], (char*)S.fld[f] - PADB));
  for (int t = 0; t < ncoef(M->kind); ++t) CK(cudaIpcGetMemHandle(&p.coef[t], (char*)coef_of(S, t) - PADB));
  CK(cudaIpcGetMemHandle(&p.flags, M->flags));
  std::memcpy(blob, &p, sizeof p);
  return SEIS_OK;
}

seis_status seis_model_peer_import(seis_model* M, const uint8_t* lo_blob, uint64_t lo_len,
                                   const uint8_t* hi_blob, uint64_t hi_len) {
  if (!M) return fail(SEIS_EINVAL, "null model");
  if (!M->comm || M->nranks < 2 || M->slabs.size() != 1)
    return fail(SEIS_EINVAL, "peer halo needs a multi-rank model (one slab per rank)");
  if (!M->flags) return fail(SEIS_EINVAL, "seis_model_peer_export must run first");
  if (M->peer) return fail(SEIS_EINVAL, "peer halo already imported");
  const bool has_lo = M->rank > 0, has_hi = M->rank < M->nranks - 1;
  if (has_lo) TRY(check_blob(M, lo_blob, lo_len, M->rank - 1));
  if (has_hi) TRY(check_blob(M, hi_blob, hi_len, M->rank + 1));
  CK(cudaSetDevice(M->device));
  TRY(memops_init());
  Slab& S = M->slabs.front();
  const size_t PS = (size_t)S.d.PS;
  for (int side = 0; side < 2; ++side) {
    if (side == 0 ? !has_lo : !has_hi) continue;
    PeerBlob p;
    std::memcpy(&p, side == 0 ? lo_blob : hi_blob, sizeof p);
    for (size_t f = 0; f < S.fld.size(); ++f) {
      char* q = nullptr;
      TRY(peer_open(M, p.fld[f], &q));
      float* rf = (float*)(q + PADB);
      if (side == 0) {  // the rank above: my planes 0..3 -> its bottom ghosts nzl_lo + k
        S.gh[f].lo = rf;
        S.gh[f].loo = (long long)p.nzl * S.d.PS;
      } else {          // the rank below: my planes nzl-4.. -> its top ghosts k - nzl
        S.gh[f].hi = rf;
        S.gh[f].hio = -(long long)S.d.nzl * S.d.PS;
      }
    }
    // coefficient ghost planes (rho / w at k+1 across the face), once, read from the peer
    for (int t = 0; t < ncoef(M->kind); ++t) {
      char* q = nullptr;
      TRY(peer_open(M, p.coef[t], &q));
      const float* rc = (const float*)(q + PADB);
      float* mine = coef_of(S, t);
      if (side == 0)
        CK(cudaMemcpy(mine + (GZ - 4) * PS, rc + (size_t)(p.nzl + GZ - 4) * PS, 4 * PS * sizeof(float),
                      cudaMemcpyDeviceToDevice));
      else
        CK(cudaMemcpy(mine + (size_t)(S.d.nzl + GZ) * PS, rc + GZ * PS, 4 * PS * sizeof(float),
                      cudaMemcpyDeviceToDevice));
    }
    char* q = nullptr;
    TRY(peer_open(M, p.flags, &q));
    if (side == 0) M->rflag_lo = (uint32_t*)q + 1;  // its "from below" word
    else M->rflag_hi = (uint32_t*)q + 0;            // its "from above" word
  }
  CK(cudaDeviceSynchronize());
  M->sig = 0;
  M->peer = true;
  return SEIS_OK;
}

seis_status seis_model_slab(const seis_model* M, int32_t* z0, int32_t* nz_local) {
  if (!M || !z0 || !nz_local) return fail(SEIS_EINVAL, "null argument");
  *z0 = M->pz0;
  *nz_local = M->pnzl;
  return SEIS_OK;
}

seis_status seis_memory_required(const seis_grid* g, seis_kind kind, const seis_shot* shot,
                                 int32_t nranks, uint64_t* bytes) {
  if (!bytes || nranks < 1) return fail(SEIS_EINVAL, "bad arguments");
  TRY(validate_grid(g, kind));
  int32_t z0, nzl;
  seis_slab_bounds(g->nz, nranks, 0, &z0, &nzl);
  const Dims d = make_dims(*g, 0, nzl);
  const double padded = (double)d.PS * (nzl + 2 * GZ) * 4.0;
  // (acoustic: 4 fields, psi_p + psi_q, split pair and fused step alike)
  int nf = nfields(kind), np = kind == SEIS_ISO ? 1 : (kind == SEIS_ACOUSTIC ? 2 : 3);  // m | kdt,rho | l2m,w,rho
  double b = (nf + np) * padded;
  double spml = 0.0;  // ISO O6b split components (6 per layer point, compact slabs)
  if (kind == SEIS_ISO && g->iso_pml && g->nb > 0)
    spml = 6.0 * 4.0 * 2.0 * g->nb * ((double)nzl * g->ny + (double)nzl * g->nx + (double)g->ny * g->nx);
  b += spml;
  if (kind != SEIS_ISO && g->nb > 0) {
    const double W = g->nb + 1;
    const double per = (2 * W * g->ny * (double)nzl + 2 * W * g->nx * (double)nzl + 2 * W * g->nx * (double)g->ny) * 4.0;
    b += per * (kind == SEIS_ACOUSTIC ? 2 : 6);
  }
  if (shot && shot->snap_period >= 1 && shot->nt >= 1) {
    const long long nsnap = (shot->nt - 1) / shot->snap_period;
    const long long c = shot->ckpt_period > 0 ? std::min<long long>(shot->ckpt_period, nsnap) : nsnap;
    const long long nckpt = nsnap > 0 && c > 0 ? (nsnap + c - 1) / c - 1 : 0;
    // checkpoint = every padded state field of the current set + the C-PML memory slabs
    double ck = (kind == SEIS_ACOUSTIC ? 4 : nf) * (padded + 128.0);
    if (kind != SEIS_ISO && g->nb > 0) {
      const double W = g->nb + 1;
      ck += (2 * W * g->ny * (double)nzl + 2 * W * g->nx * (double)nzl + 2 * W * g->nx * (double)g->ny) * 4.0 *
            (kind == SEIS_ACOUSTIC ? 2 : 6);
    }
    ck += spml;
    b += (double)c * nzl * (double)g->ny * g->nx * (shot->snap_bits == 24 ? 3.0 : 4.0) + (double)nckpt * ck;
  }
  *bytes = (uint64_t)b;
  return SEIS_OK;
}

}  // extern "C"

// ================================================================== shots
namespace {

// O6b storage index of global node (x, y, z) in slab S (the kernels' spml_idx), -1 outside
// the layers or without the split-field PML
int spml_index_host(const seis_model* M, const Slab& S, int x, int y, int z) {
  if (!S.sp) return -1;
  const int nb = M->g.nb;
  const float dt = M->g.dt;  // membership as the kernels test it: eta_d dt in fp32
  const float fx = (float)(M->eta1[0][x] * dt), fy = (float)(M->eta1[1][y] * dt), fz = (float)(M->eta1[2][z] * dt);
  if (fx == 0.0f && fy == 0.0f && fz == 0.0f) return -1;
  const int k = z - S.d.z0;
  const int nx = S.d.nx, ny = S.d.ny, nz = S.d.nz;
  if (fx != 0.0f) return (k * ny + y) * (2 * nb) + (x < nb ? x : x - (nx - 2 * nb));
  if (fy != 0.0f) return S.spx + (k * (2 * nb) + (y < nb ? y : y - (ny - 2 * nb))) * nx + x;
  return S.spx + S.spy + ((z < nb ? z : z - (nz - 2 * nb)) * ny + y) * nx + x;
}

// Replace a tracked device buffer by a larger one (the old one is freed, not kept until the
// model is destroyed).  A CUDA graph holding the old pointer is destroyed with it.
seis_status regrow(seis_model* M, float** buf, size_t* have, size_t elems) {
  if (*have >= elems) return SEIS_OK;
  if (*buf) {
    if (M->gexec) {
      cudaGraphExecDestroy(M->gexec);
      M->gexec = nullptr;
    }
    CK(cudaDeviceSynchronize());  // (no queued work may still use it)
    cudaFree(*buf);
    M->allocs.erase(std::find(M->allocs.begin(), M->allocs.end(), (void*)*buf));
    *buf = nullptr;
    *have = 0;
  }
  void* p = nullptr;
  TRY(alloc_track(M, &p, elems * sizeof(float)));
  *buf = (float*)p;
  *have = elems;
  return SEIS_OK;
}

struct ShotTables {
  std::vector<float*> owned;  // device allocations to free
};

seis_status setup_shot(seis_model* M, const seis_shot* sh, bool backward_injection,
                       cudaStream_t st) {
  const seis_grid& g = M->g;
  if (!sh) return fail(SEIS_EINVAL, "null shot");
  if (sh->nt < 1) return fail(SEIS_EINVAL, "nt must be >= 1");
  if (!sh->wavelet) return fail(SEIS_EINVAL, "null wavelet");
  if (sh->nrec < 0 || (sh->nrec > 0 && !sh->rec)) return fail(SEIS_EINVAL, "bad receiver list");
  if (sh->sx < 0 || sh->sy < 0 || sh->sz < 0 || sh->sx >= g.nx || sh->sy >= g.ny || sh->sz >= g.nz)
    return fail(SEIS_EINVAL, "source (%d,%d,%d) outside the grid", sh->sx, sh->sy, sh->sz);
  for (int r = 0; r < sh->nrec; ++r) {
    const int* p = sh->rec + 3 * r;
    if (p[0] < 0 || p[1] < 0 || p[2] < 0 || p[0] >= g.nx || p[1] >= g.ny || p[2] >= g.nz)
      return fail(SEIS_EINVAL, "receiver %d (%d,%d,%d) outside the grid", r, p[0], p[1], p[2]);
  }
  if (M->kind == SEIS_ELASTIC && (sh->rec_component < 0 || sh->rec_component > 3))
    return fail(SEIS_EINVAL, "rec_component must be 0..3");
  M->hwav = sh->wavelet;
  // the wavelet is copied to the device on every call: the source add reads s[n] there, so a
  // captured shot graph does not depend on the wavelet values (P:177 injection, O11)
  TRY(regrow(M, &M->dwav, &M->dwav_n, (size_t)sh->nt));
  CK(cudaMemcpyAsync(M->dwav, sh->wavelet, (size_t)sh->nt * sizeof(float), cudaMemcpyHostToDevice, st));
  // receiver tables are rebuilt only when the geometry changes (CUDA graphs keep pointers)
  uint64_t key = fnv1a(&sh->sx, 3 * sizeof(int32_t));
  key = fnv1a(&sh->nrec, sizeof(int32_t), key);
  if (sh->nrec) key = fnv1a(sh->rec, (size_t)sh->nrec * 3 * sizeof(int32_t), key);
  key = fnv1a(&sh->rec_component, sizeof(int32_t), key);
  key = key ? key : 1;  // (0 = "no tables yet")
  const bool fwd_same = key == M->fwd_key;
  const bool bwd_same = !backward_injection || key == M->bwd_key;
  if (!fwd_same && M->gexec) {  // the graph holds the gather tables about to be freed
    cudaGraphExecDestroy(M->gexec);
    M->gexec = nullptr;
  }
  const double h = g.h, dt = g.dt;
  auto point_scale = [&](int x, int y, int z) -> double {
    const size_t li = ((size_t)(z - M->pz0) * g.ny + y) * g.nx + x;
    const double v = M->hvp[li];
    if (M->kind == SEIS_ISO) {
      double eta = 0.0;
      if (g.nb > 0) eta = M->eta1[0][x] + M->eta1[1][y] + M->eta1[2][z];
      if (g.iso_pml && g.nb > 0 && ((float)(M->eta1[0][x] * dt) != 0.0f || (float)(M->eta1[1][y] * dt) != 0.0f ||
                                    (float)(M->eta1[2][z] * dt) != 0.0f))
        eta = M->eta1[0][x];  // O6b: the x component takes the source
      return v * v * dt * dt / (h * h * h) / (1.0 + eta * dt);  // O3
    }
    const double r = M->hrho[li];
    if (M->kind == SEIS_ACOUSTIC) return dt * r * v * v / (h * h * h);  // O8/O11
    const double s = M->hvs[li];
    const double mu = r * s * s, lam = r * (v * v - 2.0 * s * s);
    return dt * (lam + 2.0 / 3.0 * mu) / (h * h * h);  // O11 explosive
  };
  for (Slab& S : M->slabs) {
    const int z0 = S.d.z0, z1 = S.d.z0 + S.d.nzl;
    S.src_o = -1;
    if (sh->sz >= z0 && sh->sz < z1) {  // (used only by steps with with_src)
      S.src_o = S.d.at(sh->sx, sh->sy, sh->sz - z0);
      S.src_scale = (float)point_scale(sh->sx, sh->sy, sh->sz);
    }
    if (fwd_same && bwd_same) continue;
    // receivers owned by this slab
    std::vector<long long> off;
    std::vector<int> rid;
    for (int r = 0; r < sh->nrec; ++r) {
      const int* p = sh->rec + 3 * r;
      if (p[2] >= z0 && p[2] < z1) {
        off.push_back(S.d.at(p[0], p[1], p[2] - z0));
        rid.push_back(r);
      }
    }
    if (!fwd_same) {  // gather tables (forward phase)
      if (S.d_rec_off) {
        cudaFree(S.d_rec_off);
        cudaFree(S.d_rec_id);
        S.d_rec_off = nullptr;
        S.d_rec_id = nullptr;
      }
      S.nrec_own = (int)off.size();
      if (S.nrec_own > 0) {
        CK(dmalloc(&S.d_rec_off, off.size()));
        CK(dmalloc(&S.d_rec_id, rid.size()));
        CK(cudaMemcpy(S.d_rec_off, off.data(), off.size() * sizeof(long long), cudaMemcpyHostToDevice));
        CK(cudaMemcpy(S.d_rec_id, rid.data(), rid.size() * sizeof(int), cudaMemcpyHostToDevice));
      }
    }
    if (bwd_same) continue;
    for (auto& G2 : S.grp) {
      if (G2.off) {
        cudaFree(G2.off); cudaFree(G2.scale); cudaFree(G2.start); cudaFree(G2.mem); cudaFree(G2.surf);
        cudaFree(G2.sidx);
      }
      G2 = Slab::Groups{};
    }
    if (!off.empty()) {
      // merge duplicates: group receivers by node, members in receiver-index order (O12)
      std::map<long long, std::vector<int>> groups;
      for (size_t t = 0; t < off.size(); ++t) groups[off[t]].push_back(rid[t]);
      std::vector<long long> goff[2];
      std::vector<float> gsc[2];
      std::vector<int> gstart[2] = {{0}, {0}}, gmem[2], gsurf[2], gsidx[2];
      for (auto& kv : groups) {
        const int r0 = kv.second.front();
        const int* p = sh->rec + 3 * r0;
        const int ch = (p[2] - z0) / S.zc;
        const int part = (ch == 0 || ch == S.nzch - 1) ? 0 : 1;
        goff[part].push_back(kv.first);
        gsc[part].push_back((float)point_scale(p[0], p[1], p[2]));
        gsurf[part].push_back(M->g.free_surface && p[2] == 0 ? 1 : 0);
        gsidx[part].push_back(spml_index_host(M, S, p[0], p[1], p[2]));
        for (int r : kv.second) gmem[part].push_back(r);
        gstart[part].push_back((int)gmem[part].size());
      }
      for (int part = 0; part < 2; ++part) {
        Slab::Groups& G2 = S.grp[part];
        G2.n = (int)goff[part].size();
        if (G2.n == 0) continue;
        CK(dmalloc(&G2.off, goff[part].size()));
        CK(dmalloc(&G2.scale, gsc[part].size()));
        CK(dmalloc(&G2.start, gstart[part].size()));
        CK(dmalloc(&G2.mem, gmem[part].size()));
        CK(dmalloc(&G2.surf, gsurf[part].size()));
        CK(dmalloc(&G2.sidx, gsidx[part].size()));
        CK(cudaMemcpy(G2.sidx, gsidx[part].data(), gsidx[part].size() * sizeof(int), cudaMemcpyHostToDevice));
        CK(cudaMemcpy(G2.surf, gsurf[part].data(), gsurf[part].size() * sizeof(int), cudaMemcpyHostToDevice));
        CK(cudaMemcpy(G2.off, goff[part].data(), goff[part].size() * sizeof(long long), cudaMemcpyHostToDevice));
        CK(cudaMemcpy(G2.scale, gsc[part].data(), gsc[part].size() * sizeof(float), cudaMemcpyHostToDevice));
        CK(cudaMemcpy(G2.start, gstart[part].data(), gstart[part].size() * sizeof(int), cudaMemcpyHostToDevice));
        CK(cudaMemcpy(G2.mem, gmem[part].data(), gmem[part].size() * sizeof(int), cudaMemcpyHostToDevice));
      }
    }
  }
  M->fwd_key = key;
  if (backward_injection) M->bwd_key = key;
  M->shot_key = key;
  return SEIS_OK;
}

// Zero the state of every slab (fields incl. ghosts, C-PML slabs).
seis_status zero_state(seis_model* M, cudaStream_t st) {
  TRY(peer_barrier(M, st));  // (f4) no neighbour store into these ghost planes is in flight
  for (Slab& S : M->slabs) {
    const size_t elems = (size_t)S.d.PS * (S.d.nzl + 2 * GZ);
    for (float* f : S.fld) CK(cudaMemsetAsync(f, 0, elems * sizeof(float), st));
    if (S.sp) CK(cudaMemsetAsync(S.sp, 0, (size_t)S.spn * 6 * sizeof(float), st));
    if (M->W > 0) {
      const int W = M->W;
      const int npsi = npsi_of(M->kind);
      for (int t = 0; t < npsi; ++t) {
        const int ax = psi_axis(M->kind, t);
        size_t n;
        if (ax == 0) n = (size_t)S.d.nzl * S.d.ny * 2 * W;
        else if (ax == 1) n = (size_t)S.d.nzl * 2 * W * S.d.nx;
        else n = (size_t)2 * W * S.d.ny * S.d.nx;
        CK(cudaMemsetAsync(S.psi[t], 0, n * sizeof(float), st));
      }
    }
    S.cur = 0;
  }
  return peer_barrier(M, st);  // (f4) ... nor starts before the reset is done
}

// Every array of the propagating state (padded fields incl. ghost planes, C-PML
// memory slabs): (pointer, floats).  A checkpoint is a copy of all of them.
std::vector<std::pair<float*, size_t>> state_arrays(seis_model* M) {
  std::vector<std::pair<float*, size_t>> v;
  for (Slab& S : M->slabs) {
    const size_t elems = (size_t)S.d.PS * (S.d.nzl + 2 * GZ) + 32;  // + the 128-byte alignment pad
    for (size_t f = 0; f < S.fld.size(); ++f) v.emplace_back(S.fld[f] - 28, elems);  // base = f - 112 bytes
    if (S.sp) v.emplace_back(S.sp, (size_t)S.spn * 6);  // ISO O6b split components
    if (M->W > 0) {
      const int W = M->W;
      for (int t = 0; t < npsi_of(M->kind); ++t) {
        const int ax = psi_axis(M->kind, t);
        size_t n;
        if (ax == 0) n = (size_t)S.d.nzl * S.d.ny * 2 * W;
        else if (ax == 1) n = (size_t)S.d.nzl * 2 * W * S.d.nx;
        else n = (size_t)2 * W * S.d.ny * S.d.nx;
        v.emplace_back(S.psi[t], n);
      }
    }
  }
  return v;
}

// Copy the whole state to (save = true) or from a checkpoint slot of state_elems floats.
seis_status state_copy(seis_model* M, float* slot, bool save, cudaStream_t st) {
  TRY(peer_barrier(M, st));  // (f4) the ghost planes are settled (see zero_state)
  size_t o = 0;
  for (auto& a : state_arrays(M)) {
    if (save) CK(cudaMemcpyAsync(slot + o, a.first, a.second * 4, cudaMemcpyDeviceToDevice, st));
    else CK(cudaMemcpyAsync(a.first, slot + o, a.second * 4, cudaMemcpyDeviceToDevice, st));
    o += (a.second + 31) / 32 * 32;
  }
  return peer_barrier(M, st);
}
size_t state_elems(seis_model* M) {
  size_t o = 0;
  for (auto& a : state_arrays(M)) o += (a.second + 31) / 32 * 32;
  return o;
}


// ISO / ACOUSTIC: 64 x BY tiles of (16, BY) threads; ELASTIC: 32 x BYE tiles of (32, BYE)
dim3 grid_of(const Slab& S, int tw, int by, int nch) {
  return dim3((S.d.nx + tw - 1) / tw, (S.d.ny + by - 1) / by, nch);
}

// Backward-phase receiver injection into the field just produced (before its
// ghost planes are exchanged, so neighbouring slabs see the injected values).
// part: 0 = groups in the first / last z-chunk, 1 = interior chunks, 2 = all.
seis_status inject_rows(seis_model* M, const float* row, int part, cudaStream_t st) {
  for (Slab& S : M->slabs) {
    for (int q = 0; q < 2; ++q) {
      if (part != 2 && part != q) continue;
      const Slab::Groups& G2 = S.grp[q];
      if (G2.n == 0) continue;
      PROF(5, st);
      if (M->kind == SEIS_ELASTIC) {
        inject_el_kernel<<<(G2.n + 127) / 128, 128, 0, st>>>(S.fld[ESXX], S.fld[ESYY], S.fld[ESZZ], G2.off,
                                                            G2.scale, G2.start, G2.mem, row, G2.surf, G2.n,
                                                            S.gh[ESZZ], S.d.PS, S.d.nzl);
      } else {
        const int f = M->kind == SEIS_ISO ? S.cur : 0;
        inject_kernel<<<(G2.n + 127) / 128, 128, 0, st>>>(S.fld[f], G2.off, G2.scale, G2.start, G2.mem, row,
                                                         G2.n, S.gh[f], S.d.PS, S.d.nzl, G2.sidx,
                                                         S.sp ? S.sp + (size_t)S.cur * 3 * S.spn : nullptr);
      }
      CKL();
    }
  }
  return SEIS_OK;
}

// Launch of one stencil kernel on slab s over the z-chunks ch0 + t chs, t < nch.
using LaunchFn = std::function<seis_status(size_t s, int ch0, int chs, int nch, cudaStream_t)>;
// Work after the kernel: part 0 = first/last chunks (injection there, then the ghost
// exchange and free-surface mirror), part 1 = interior chunks, part 2 = everything.
using PostFn = std::function<seis_status(int part, cudaStream_t)>;

// Is the ghost exchange of this model overlapped with interior updates?
bool overlapped(const seis_model* M) {
  if (M->slabs.size() < 2 && !(M->comm && M->nranks > 1)) return false;  // nothing to exchange
  return !M->no_overlap;
}

// One kernel phase of a step (8(e) pipeline).  Without decomposition: every chunk, then
// `post(2)`.  Decomposed: the first and last z-chunk of every slab run first on the side
// stream xs, followed there by their injection, the ghost-plane exchange (memcpy between
// slabs, NCCL send/recv between ranks) and the mirror; meanwhile the interior chunks run on
// the compute stream; the compute stream then joins xs.  Per-point arithmetic is the same,
// so results are bitwise identical to the serial order.
//
// f4 (M->peer): the boundary chunks read ghost planes the neighbour ranks store directly, so
// they wait for the neighbours' signal of the previous phase; after them (and the injection
// of their nodes) this rank signals in turn.  Interior chunks touch no ghost plane.  The
// write-after-read order on the ghosts needs no extra signal: a neighbour stores into my
// ghosts of field F only after waiting for my signal of the phase that READ them (every
// boundary-chunk kernel reads the ghosts of the previous phase's field and stores those of
// its own).
seis_status run_phase(seis_model* M, const LaunchFn& launch, const PostFn& post, cudaStream_t st) {
  if (!overlapped(M)) {
    TRY(peer_wait(M, st));
    for (size_t s = 0; s < M->slabs.size(); ++s) TRY(launch(s, 0, 1, M->slabs[s].nzch, st));
    TRY(post(2, st));
    return peer_signal(M, st);
  }
  cudaStream_t xs = M->xs;
  CK(cudaEventRecord(M->ev_fork, st));
  CK(cudaStreamWaitEvent(xs, M->ev_fork, 0));
  TRY(peer_wait(M, xs));
  for (size_t s = 0; s < M->slabs.size(); ++s) {
    const int nch = M->slabs[s].nzch;
    if (nch <= 2) TRY(launch(s, 0, 1, nch, xs));
    else TRY(launch(s, 0, nch - 1, 2, xs));
  }
  TRY(post(0, xs));
  TRY(peer_signal(M, xs));
  for (size_t s = 0; s < M->slabs.size(); ++s) {
    const int nch = M->slabs[s].nzch;
    if (nch > 2) TRY(launch(s, 1, 1, nch - 2, st));
  }
  TRY(post(1, st));
  CK(cudaEventRecord(M->ev_join, xs));
  CK(cudaStreamWaitEvent(st, M->ev_join, 0));
  return SEIS_OK;
}

// One forward time step of every slab of the process, incl. exchanges.
//   snap: compact snapshot target per slab (or null), imgS/img: imaging of the INPUT level,
//   inj_row: receiver samples injected into the produced field (backward phase) or null
seis_status step(seis_model* M, int n, bool with_src, std::vector<float*>* snap,
                 std::vector<SnapRef>* imgS, std::vector<float*>* img, cudaStream_t st,
                 const float* inj_row = nullptr) {
  auto inject = [&](int part, cudaStream_t s2) -> seis_status {
    return inj_row ? inject_rows(M, inj_row, part, s2) : SEIS_OK;
  };
  if (M->kind == SEIS_ISO) {
    const int cur = M->slabs[0].cur;  // u^n = fld[cur] in every slab
    LaunchFn k_iso = [&](size_t s, int ch0, int chs, int nch, cudaStream_t ks) -> seis_status {
      Slab& S = M->slabs[s];
      IsoArgs a;
      a.mun = S.iso_ut[cur];
      a.mup = S.iso_uc[1 - cur];
      a.mm = S.iso_m;
      a.muq = S.iso_uc[cur];
      a.un = S.fld[cur];
      a.up = S.fld[1 - cur];
      a.edx = M->edx;
      a.edy = M->edy;
      a.edz = M->edz;
      a.d = S.d;
      a.zc = S.zc;
      a.ch0 = ch0;
      a.chs = chs;
      a.src_o = with_src ? S.src_o : -1;
      a.src = SrcAmp{M->dwav, n, S.src_scale};
      a.snap = snap ? (*snap)[s] : nullptr;
      a.imgS = imgS ? (*imgS)[s].s32 : nullptr;
      if (imgS) a.imgR = (*imgS)[s];
      a.img = img ? (*img)[s] : nullptr;
      a.gh = S.gh[1 - cur];
      a.sp = S.sp;
      a.spn = S.spn;
      a.nbl = M->g.nb;
      a.nxs = S.spx;
      a.nys = S.spy;
      a.lvl = cur;
      for (int t = 0; t < 3; ++t) {
        a.spco[t] = M->spco[t];
        a.spnp[t] = M->spnp[t];
      }
      const dim3 gr = grid_of(S, TXV, BYI, nch), blk(NTX, BYI);
      {
        PROF(0, ks);
        // template flags: O6b split-field PML; direct ghost stores of this slab (f4)
        auto go = [&](auto spml, auto gh) {
          constexpr bool SP = decltype(spml)::value, GH = decltype(gh)::value;
          const size_t sb = SP ? IsoStage<BYI>::smem_bytes_spml() : IsoStage<BYI>::smem_bytes();
          if (a.snap) iso_step_kernel<BYI, true, false, SP, GH><<<gr, blk, sb, ks>>>(a);
          else if (a.img) iso_step_kernel<BYI, false, true, SP, GH><<<gr, blk, sb, ks>>>(a);
          else iso_step_kernel<BYI, false, false, SP, GH><<<gr, blk, sb, ks>>>(a);
        };
        const bool gh = a.gh.lo || a.gh.hi;
        a.region = 0;
        a.nbr = M->g.nb;
        if (S.sp) {
          // O6b: the blocks without layer points run the plain kernel (96 registers, high
          // occupancy), the others the split-field kernel; disjoint points, same arithmetic for
          // the non-layer points of either.  The two launches run concurrently (the plain one
          // on a side stream) so the light blocks fill the SMs around the heavy ones.
          static const bool conc = !(getenv("SEIS_SPML_CONC") && getenv("SEIS_SPML_CONC")[0] == '0');
          if (conc && !M->sps) {
            CK(cudaStreamCreateWithFlags(&M->sps, cudaStreamNonBlocking));
            CK(cudaEventCreateWithFlags(&M->ev_spf, cudaEventDisableTiming));
            CK(cudaEventCreateWithFlags(&M->ev_spj, cudaEventDisableTiming));
          }
          cudaStream_t ks2 = ks;
          if (conc) {
            CK(cudaEventRecord(M->ev_spf, ks));
            CK(cudaStreamWaitEvent(M->sps, M->ev_spf, 0));
          }
          a.region = 2;
          if (gh) go(std::true_type{}, std::true_type{});
          else go(std::true_type{}, std::false_type{});
          a.region = 1;
          if (conc) ks = M->sps;
          if (gh) go(std::false_type{}, std::true_type{});
          else go(std::false_type{}, std::false_type{});
          ks = ks2;
          if (conc) {
            CK(cudaEventRecord(M->ev_spj, M->sps));
            CK(cudaStreamWaitEvent(ks, M->ev_spj, 0));
          }
          ++g_launches;  // two launches (CKL counts one)
        } else if (gh) go(std::false_type{}, std::true_type{});
        else go(std::false_type{}, std::false_type{});
      }
      CKL();
      return SEIS_OK;
    };
    // the injection targets u^{n+1} = fld[1 - cur]; swap first so inject_rows sees it as cur
    for (Slab& S : M->slabs) S.cur = 1 - S.cur;
    PostFn post = [&](int part, cudaStream_t ps) -> seis_status {
      TRY(inject(part, ps));
      if (part != 1) TRY(exchange(M, {1 - cur}, ps));  // the new level
      return SEIS_OK;
    };
    return run_phase(M, k_iso, post, st);
  }
  if (M->kind == SEIS_ACOUSTIC && M->ac_step) {
    // f1: the whole step (V then P) in one persistent launch (kernels_acoustic_step.cuh); one
    // slab, no exchange.  Cooperative launch: every tile's CTA is resident (they wait on their
    // neighbours' progress counters, which the memset zeroes first).
    Slab& S = M->slabs[0];
    AcSArgs a;
    a.mpt = S.as_pt;
    a.mqx = S.as_q[0];
    a.mqy = S.as_q[1];
    a.mqz = S.as_q[2];
    a.mrt = S.as_rt;
    a.mrz = S.as_rz;
    a.mpq = S.as_pq;
    a.mqxn = S.as_qxn;
    a.mqyn = S.as_qyn;
    a.mk = S.as_k;
    a.p0 = S.fld[0];
    a.p = S.fld[0];
    a.qx = S.fld[1];
    a.qy = S.fld[2];
    a.qz = S.fld[3];
    a.kk = S.kdt;
    a.dth = (float)((double)M->g.dt / (double)M->g.h);
    a.W = M->W;
    a.zlo = 1;
    a.cx = M->cp[0];
    a.cy = M->cp[1];
    a.cz = M->cp[2];
    a.psx = S.psi[0];
    a.psy = S.psi[1];
    a.psz = S.psi[2];
    a.pqx = S.psi[3];
    a.pqy = S.psi[4];
    a.pqz = S.psi[5];
    a.d = S.d;
    a.ntx = M->as_ntx;
    a.nty = M->as_nty;
    a.cnt = M->as_cnt;
    a.src_o = with_src ? S.src_o : -1;
    a.src = SrcAmp{M->dwav, n, S.src_scale};
    a.snap = snap ? (*snap)[0] : nullptr;
    if (imgS) a.imgR = (*imgS)[0];
    a.img = img ? (*img)[0] : nullptr;
    a.trace = nullptr;
#if SEIS_AS_TRACE
    {
      static unsigned long long* tr = nullptr;
      static size_t trn = 0;
      const size_t need = (size_t)M->as_ntx * M->as_nty * S.d.nzl * 48;
      if (trn < need) {
        if (tr) cudaFree(tr);
        CK(cudaMallocManaged(&tr, need * sizeof(unsigned long long)));
        trn = need;
      }
      a.trace = tr;
      g_trace = tr;
      g_trace_n = need;
    }
#endif
    const int ntiles = M->as_ntx * M->as_nty;
    CK(cudaMemsetAsync(M->as_cnt, 0, (size_t)ntiles * sizeof(unsigned), st));
    {
      PROF(9, st);
      cudaLaunchConfig_t cfg = {};
      cfg.gridDim = dim3(ntiles);
      cfg.blockDim = dim3(AS_THREADS);
      cfg.dynamicSmemBytes = AcSLayout::smem_bytes();
      cfg.stream = st;
      cudaLaunchAttribute attr[1];
      attr[0].id = cudaLaunchAttributeCooperative;
      attr[0].val.cooperative = 1;
      cfg.attrs = attr;
      cfg.numAttrs = 1;
      if (a.snap) CK(cudaLaunchKernelEx(&cfg, ac_step_kernel<true, false>, a));
      else if (a.img) CK(cudaLaunchKernelEx(&cfg, ac_step_kernel<false, true>, a));
      else CK(cudaLaunchKernelEx(&cfg, ac_step_kernel<false, false>, a));
    }
    CKL();
    return inj_row ? inject_rows(M, inj_row, 2, st) : SEIS_OK;
  }
  if (M->kind == SEIS_ACOUSTIC) {
    LaunchFn k_v = [&](size_t s, int ch0, int chs, int nch, cudaStream_t ks) -> seis_status {
      Slab& S = M->slabs[s];
      AcVArgs a;
      a.mp = S.ac_pt;
      a.mqx = S.ac_qc[0];
      a.mqy = S.ac_qc[1];
      a.mqz = S.ac_qc[2];
      a.mr = S.ac_rt;
      a.mpq = S.ac_pc;
      a.mrz = S.ac_rc;
      a.p = S.fld[0];
      a.rho = S.rho;
      a.dth = (float)((double)M->g.dt / (double)M->g.h);
      a.qx = S.fld[1];
      a.qy = S.fld[2];
      a.qz = S.fld[3];
      a.W = M->W;
      a.zlo = 1;
      a.cx = M->cp[0];
      a.cy = M->cp[1];
      a.cz = M->cp[2];
      a.psx = S.psi[0];
      a.psy = S.psi[1];
      a.psz = S.psi[2];
      a.d = S.d;
      a.zc = S.zc;
      a.ch0 = ch0;
      a.chs = chs;
      a.imgS = imgS ? (*imgS)[s].s32 : nullptr;
      if (imgS) a.imgR = (*imgS)[s];
      a.img = img ? (*img)[s] : nullptr;
      a.gh = S.gh[3];
      const dim3 gr = grid_of(S, TXV, BYV, nch), blk(NTX, BYV);
      {
        PROF(1, ks);
        const size_t sb = AcVStage<BYV>::smem_bytes();
        if (a.img) ac_v_kernel<BYV, true><<<gr, blk, sb, ks>>>(a);
        else ac_v_kernel<BYV, false><<<gr, blk, sb, ks>>>(a);
      }
      CKL();
      return SEIS_OK;
    };
    // q_z has the only z-derivative in P
    TRY(run_phase(M, k_v, [&](int part, cudaStream_t ps) { return part != 1 ? exchange(M, {3}, ps) : SEIS_OK; },
                  st));
    LaunchFn k_p = [&](size_t s, int ch0, int chs, int nch, cudaStream_t ks) -> seis_status {
      Slab& S = M->slabs[s];
      AcPArgs a;
      a.mqx = S.ac_qxt;
      a.mqy = S.ac_qyt;
      a.mpp = S.ac_ppc;
      a.mk = S.ac_kc;
      a.mqq = S.ac_qzc;
      a.p = S.fld[0];
      a.qz = S.fld[3];
      a.W = M->W;
      a.zlo = 1;
      a.cx = M->cp[0];
      a.cy = M->cp[1];
      a.cz = M->cp[2];
      a.pqx = S.psi[3];
      a.pqy = S.psi[4];
      a.pqz = S.psi[5];
      a.d = S.d;
      a.zc = S.zc;
      a.ch0 = ch0;
      a.chs = chs;
      a.src_o = with_src ? S.src_o : -1;
      a.src = SrcAmp{M->dwav, n, S.src_scale};
      a.snap = snap ? (*snap)[s] : nullptr;
      a.gh = S.gh[0];
      const dim3 gr = grid_of(S, TXV, BYP, nch), blk(NTX, BYP);
      {
        PROF(2, ks);
        const size_t sb = AcPStage<BYP>::smem_bytes();
        if (a.snap) ac_p_kernel<BYP, true><<<gr, blk, sb, ks>>>(a);
        else ac_p_kernel<BYP, false><<<gr, blk, sb, ks>>>(a);
      }
      CKL();
      return SEIS_OK;
    };
    PostFn post_p = [&](int part, cudaStream_t ps) -> seis_status {
      TRY(inject(part, ps));
      if (part != 1) TRY(exchange(M, {0}, ps));  // p for the next V
      return SEIS_OK;
    };
    return run_phase(M, k_p, post_p, st);
  }
  // ELASTIC
  LaunchFn k_v = [&](size_t s, int ch0, int chs, int nch, cudaStream_t ks) -> seis_status {
    Slab& S = M->slabs[s];
    ElVArgs a;
    a.msxx = S.el_sxxt;
    a.msxy = S.el_sxyt;
    a.msxz = S.el_sxzt;
    a.msyy = S.el_syyt;
    a.msyz = S.el_syzt;
    a.mr = S.el_rt;
    a.mrz = S.el_rc;
    a.dth = (float)((double)M->g.dt / (double)M->g.h);
    for (int t = 0; t < 3; ++t) {
      a.mv[t] = S.el_vc[t];
    }
    a.mq[0] = S.el_sc[ESXZ - ESXX];
    a.mq[1] = S.el_sc[ESYZ - ESXX];
    a.mq[2] = S.el_sc[ESZZ - ESXX];
    for (int t = 0; t < 9; ++t) a.f[t] = S.fld[t];
    a.W = M->W;
    a.zlo = M->g.free_surface ? 0 : 1;
    a.fs = M->g.free_surface;
    a.cx = M->cp[0];
    a.cy = M->cp[1];
    a.cz = M->cp[2];
    for (int t = 0; t < 9; ++t) a.psi[t] = S.psi[t];
    a.d = S.d;
    a.zc = S.zc;
    a.ch0 = ch0;
    a.chs = chs;
    a.imgS = imgS ? (*imgS)[s].s32 : nullptr;
    if (imgS) a.imgR = (*imgS)[s];
    a.img = img ? (*img)[s] : nullptr;
    for (int t = 0; t < 3; ++t) a.gh[t] = S.gh[EVX + t];
    const dim3 gr = grid_of(S, TXE, BYE, nch);
    {
      PROF(3, ks);
      auto go = [&](auto cp) {
        constexpr bool CP = decltype(cp)::value;
        if (a.img) el_v_kernel<BYE, true, CP><<<gr, dim3(NTX2, BYE + EL_WS), ElVStage<BYE>::smem_bytes(), ks>>>(a);
        else el_v_kernel<BYE, false, CP><<<gr, dim3(NTX2, BYE + EL_WS), ElVStage<BYE>::smem_bytes(), ks>>>(a);
      };
      el_regions(a.region, a.W, go);
    }
    CKL();
    return SEIS_OK;
  };
  PostFn post_v = [&](int part, cudaStream_t ps) -> seis_status {
    if (part == 1) return SEIS_OK;
    return exchange(M, {0, 1, 2}, ps);  // (free-surface images: formed in el_s's z-queue warm-up)
  };
  TRY(run_phase(M, k_v, post_v, st));
  LaunchFn k_s = [&](size_t s, int ch0, int chs, int nch, cudaStream_t ks) -> seis_status {
    Slab& S = M->slabs[s];
    ElSArgs a;
    for (int t = 0; t < 3; ++t) a.mvt[t] = S.el_vt[t];
    for (int t = 0; t < 6; ++t) a.ms[t] = S.el_sc[t];
    a.ml2m = S.el_l2m;
    a.mw = S.el_w;
    for (int t = 0; t < 3; ++t) a.mq[t] = S.el_vc[t];
    for (int t = 0; t < 9; ++t) a.f[t] = S.fld[t];
    a.W = M->W;
    a.zlo = M->g.free_surface ? 0 : 1;
    a.fs = M->g.free_surface;
    a.cx = M->cp[0];
    a.cy = M->cp[1];
    a.cz = M->cp[2];
    for (int t = 0; t < 9; ++t) a.psi[t] = S.psi[9 + t];
    a.d = S.d;
    a.zc = S.zc;
    a.ch0 = ch0;
    a.chs = chs;
    a.src_o = with_src ? S.src_o : -1;
    a.src = SrcAmp{M->dwav, n, S.src_scale};
    a.snap = snap ? (*snap)[s] : nullptr;
    a.gh[0] = S.gh[ESZZ];
    a.gh[1] = S.gh[ESXZ];
    a.gh[2] = S.gh[ESYZ];
    const dim3 gr = grid_of(S, TXE, BYE, nch);
    {
      PROF(4, ks);
      auto go = [&](auto cp) {
        constexpr bool CP = decltype(cp)::value;
        if (a.snap) el_s_kernel<BYE, true, CP><<<gr, dim3(NTX2, BYE + EL_WS), ElSStage<BYE>::smem_bytes(), ks>>>(a);
        else el_s_kernel<BYE, false, CP><<<gr, dim3(NTX2, BYE + EL_WS), ElSStage<BYE>::smem_bytes(), ks>>>(a);
      };
      el_regions(a.region, a.W, go);
    }
    CKL();
    return SEIS_OK;
  };
  PostFn post_s = [&](int part, cudaStream_t ps) -> seis_status {
    TRY(inject(part, ps));
    if (part == 1) return SEIS_OK;
    return exchange(M, {5, 7, 8}, ps);  // (free-surface images: formed in el_v's z-queue warm-up)
  };
  return run_phase(M, k_s, post_s, st);
}

// f1: ISO time steps n and n + 1 in one cooperative launch (kernels_iso2.cuh); u^{n+1} lands
// in fld[1 - cur], u^{n+2} in fld[cur] (cur is unchanged, as after two single steps).
seis_status step2(seis_model* M, int n, cudaStream_t st) {
  Slab& S = M->slabs[0];
  const int c = S.cur;
  Iso2Args a;
  a.mat = S.i2_t[c];
  a.mbc = S.i2_c[1 - c];
  a.mm = S.i2_m;
  a.mac = S.i2_c[c];
  a.mbt = S.i2_t[1 - c];
  a.ua = S.fld[c];
  a.ub = S.fld[1 - c];
  a.uaw = S.fld[c];
  a.edx = M->edx;
  a.edy = M->edy;
  a.edz = M->edz;
  a.d = S.d;
  a.ntx = M->i2_ntx;
  a.nty = M->i2_nty;
  a.cnt = M->i2_cnt;
  a.src_o = S.src_o;
  a.src1 = SrcAmp{M->dwav, n, S.src_scale};
  a.src2 = SrcAmp{M->dwav, n + 1, S.src_scale};
  const int ntiles = M->i2_ntx * M->i2_nty;
  CK(cudaMemsetAsync(M->i2_cnt, 0, (size_t)ntiles * sizeof(unsigned), st));
  {
    PROF(10, st);
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(ntiles);
    cfg.blockDim = dim3(I2_THREADS);
    cfg.dynamicSmemBytes = Iso2Layout::smem_bytes();
    cfg.stream = st;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeCooperative;
    attr[0].val.cooperative = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    if (a.edx) CK(cudaLaunchKernelEx(&cfg, iso2_kernel<true>, a));
    else CK(cudaLaunchKernelEx(&cfg, iso2_kernel<false>, a));
  }
  CKL();
  return SEIS_OK;
}

// Field holding the recorded / imaged quantity
const float* out_field(seis_model* M, Slab& S, int comp) {
  if (M->kind == SEIS_ISO) return S.fld[S.cur];
  if (M->kind == SEIS_ACOUSTIC) return S.fld[0];
  if (comp == 3) return S.fld[3];
  return S.fld[comp];
}

seis_status gather(seis_model* M, const seis_shot* sh, float* seis_dev, int n, cudaStream_t st) {
  for (Slab& S : M->slabs) {
    if (S.nrec_own == 0) continue;
    const int comp = M->kind == SEIS_ELASTIC ? sh->rec_component : 0;
    const float* f0 = out_field(M, S, comp);
    const int pres = (M->kind == SEIS_ELASTIC && comp == 3);
    PROF(6, st);
    gather_kernel<<<(S.nrec_own + 127) / 128, 128, 0, st>>>(
        seis_dev + (size_t)n * sh->nrec, f0, pres ? S.fld[4] : f0, pres ? S.fld[5] : f0,
        S.d_rec_off, S.d_rec_id, S.nrec_own, pres);
    CKL();
  }
  return SEIS_OK;
}

seis_status ensure_stage(seis_model* M, size_t elems) { return regrow(M, &M->stage, &M->stage_elems, elems); }

}  // namespace

// Small L2-resident ISO grids: the whole shot as one cooperative launch -- resident bricks
// (iso_resident_kernel) where they fit, else the grid-stride kernel (iso_persist_kernel).
bool persist_ok(const seis_model* M) {
  if (M->kind != SEIS_ISO || M->slabs.size() != 1 || M->comm || prof::on) return false;
  const Slab& S = M->slabs[0];
  if (S.sp) return false;  // (the split-field PML keeps the z-march kernel)
  const char* e = getenv("SEIS_NO_PERSIST");
  const bool off = e && e[0] == '1';
  return !off && (double)S.d.nx * S.d.ny * S.d.nzl < 4.0 * 1024 * 1024;
}

seis_status forward_persist(seis_model* M, const seis_shot* sh, float* sd, size_t ns, cudaStream_t st) {
  Slab& S = M->slabs[0];
  TRY(zero_state(M, st));
  if (ns) CK(cudaMemsetAsync(sd, 0, ns * sizeof(float), st));
  IsoPArgs a;
  a.u0 = S.fld[0];
  a.u1 = S.fld[1];
  a.m = S.m;
  a.edx = M->edx;
  a.edy = M->edy;
  a.edz = M->edz;
  a.d = S.d;
  a.nt = sh->nt;
  a.cur0 = S.cur;
  a.src_o = S.src_o;
  a.w = M->dwav;
  a.src_scale = S.src_scale;
  a.seis = sd;
  a.rec_off = S.d_rec_off;
  a.rec_id = S.d_rec_id;
  a.nrec = S.nrec_own;
  a.nrec_tot = sh->nrec;
  static int occ = 0, nsm = 0, rocc64 = 0, rocc128 = 0;
  if (!occ) {
    CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, iso_persist_kernel, 128, 0));
    CK(cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, M->device));
    CK(cudaFuncSetAttribute(iso_resident_kernel<64>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                            (int)IrShape<64>::smem()));
    CK(cudaFuncSetAttribute(iso_resident_kernel<128>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                            (int)IrShape<128>::smem()));
    CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&rocc64, iso_resident_kernel<64>, IrShape<64>::THREADS,
                                                     IrShape<64>::smem()));
    CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&rocc128, iso_resident_kernel<128>, IrShape<128>::THREADS,
                                                     IrShape<128>::smem()));
  }
  // Resident bricks (iso_resident_kernel) when nx <= 128, every brick gets its own co-resident
  // CTA and the receivers fit the per-brick list; else the grid-stride kernel with grid
  // barriers.  SEIS_ISO_RESIDENT=0 forces the latter (comparison), =2 requires the former.
  const int tx = S.d.nx <= 64 ? 64 : 128;
  const int nby = (S.d.ny + IR_TY - 1) / IR_TY, nbz = (S.d.nzl + IR_TZ - 1) / IR_TZ;
  const long long bricks = (long long)nby * nbz;
  const int rocc = tx == 64 ? rocc64 : rocc128;
  const char* er = getenv("SEIS_ISO_RESIDENT");
  const bool fits = S.d.nx <= 128 && bricks <= (long long)rocc * nsm && sh->nrec <= IR_RECMAX;
  if (er && er[0] == '2' && !fits)
    return fail(SEIS_EINVAL, "resident ISO kernel: nx %d > 128, %lld bricks > %d co-resident CTAs, or %d receivers > %d",
                S.d.nx, bricks, rocc * nsm, sh->nrec, IR_RECMAX);
  if (!(er && er[0] == '0') && fits) {
    const size_t xbytes = (size_t)bricks * 2 * (tx * IR_TY * IR_TZ / 2) * 16;
    if (M->rxb_n != xbytes) {  // (a model's grid is fixed: allocated and zeroed once)
      void* p = nullptr;
      TRY(alloc_track(M, &p, xbytes));
      M->rxb = p;
      M->rxb_n = xbytes;
      M->rxb_base = 0;
      CK(cudaMemsetAsync(M->rxb, 0, xbytes, st));
    }
    IsoRArgs r;
    r.u0 = S.fld[0];
    r.u1 = S.fld[1];
    r.m = S.m;
    r.edx = M->edx;
    r.edy = M->edy;
    r.edz = M->edz;
    r.d = S.d;
    r.nt = sh->nt;
    r.cur0 = S.cur;
    r.src_o = S.src_o;
    r.w = M->dwav;
    r.src_scale = S.src_scale;
    r.seis = sd;
    r.rec_off = S.d_rec_off;
    r.rec_id = S.d_rec_id;
    r.nrec = S.nrec_own;
    r.nrec_tot = sh->nrec;
    r.xb = (uint4*)M->rxb;
    r.base = M->rxb_base;
    r.nby = nby;
    r.nbz = nbz;
    r.trace = nullptr;
#if SEIS_AS_TRACE
    {
      static unsigned long long* tr = nullptr;
      static size_t trn = 0;
      const size_t need = (size_t)bricks * sh->nt * 4;
      if (trn < need) {
        if (tr) cudaFree(tr);
        CK(cudaMallocManaged(&tr, need * sizeof(unsigned long long)));
        trn = need;
      }
      r.trace = tr;
      g_trace = tr;
      g_trace_n = need;
    }
#endif
    void* rargs[] = {&r};
    if (tx == 64)
      CK(cudaLaunchCooperativeKernel((void*)iso_resident_kernel<64>, dim3((unsigned)bricks),
                                     dim3(IrShape<64>::THREADS), rargs, IrShape<64>::smem(), st));
    else
      CK(cudaLaunchCooperativeKernel((void*)iso_resident_kernel<128>, dim3((unsigned)bricks),
                                     dim3(IrShape<128>::THREADS), rargs, IrShape<128>::smem(), st));
    ++g_launches;
    M->rxb_base += (unsigned)sh->nt;
    S.cur = (S.cur + sh->nt) & 1;
    return SEIS_OK;
  }
  const long long groups = (long long)((S.d.nx + 3) / 4) * S.d.ny * S.d.nzl;
  const char* eb = getenv("SEIS_PERSIST_BPSM");  // blocks per SM (A/B; default: all that fit)
  const int bpsm = eb ? std::max(1, std::min(atoi(eb), occ)) : occ;
  const int blocks = (int)std::max<long long>(1, std::min<long long>((groups + 127) / 128, (long long)bpsm * nsm));
  void* args[] = {&a};
  CK(cudaLaunchCooperativeKernel((void*)iso_persist_kernel, dim3(blocks), dim3(128), args, 0, st));
  ++g_launches;
  S.cur = (S.cur + sh->nt) & 1;  // the z-march path's final level bookkeeping
  return SEIS_OK;
}

extern "C" {

// The time loop of one modeling shot (everything between the zeroed state and the
// filled seismogram), issued on `st`.
static seis_status forward_loop(seis_model* M, const seis_shot* sh, float* sd, size_t ns, cudaStream_t st) {
  TRY(zero_state(M, st));
  if (ns) CK(cudaMemsetAsync(sd, 0, ns * sizeof(float), st));
  for (int n = 0; n < sh->nt;) {
    if (M->iso2 && n + 1 < sh->nt) {  // steps n, n + 1 in one launch (f1), then both rows
      if (prof::sample > 1) prof::sample_now = n % prof::sample == 0 || (n + 1) % prof::sample == 0;
      TRY(step2(M, n, st));
      if (sh->nrec) {
        Slab& S = M->slabs[0];
        const int c0 = S.cur;  // u^{n+1} is in fld[1 - c0], u^{n+2} in fld[c0]
        S.cur = 1 - c0;
        TRY(gather(M, sh, sd, n, st));
        S.cur = c0;
        TRY(gather(M, sh, sd, n + 1, st));
      }
      n += 2;
      continue;
    }
    if (prof::sample > 1) prof::sample_now = n % prof::sample == 0;
    TRY(step(M, n, true, nullptr, nullptr, nullptr, st));
    if (sh->nrec) TRY(gather(M, sh, sd, n, st));
    ++n;
  }
  prof::sample_now = true;
  // (a peer-only communicator has no NCCL: each rank returns its own receivers' columns; a
  // 1-rank NCCL communicator runs the same all-reduce, an identity)
  if (M->comm && M->comm->nccl && ns)
    NK(ncclAllReduce(sd, sd, ns, ncclFloat, ncclSum, M->comm->nccl, st));
  return SEIS_OK;
}

seis_status seis_forward_model(seis_model* M, const seis_shot* sh, float* seis, void* stream) {
  g_launches = 0;
  if (!M) return fail(SEIS_EINVAL, "null model");
  if (!seis && sh && sh->nrec > 0) return fail(SEIS_EINVAL, "null seis");
  CK(cudaSetDevice(M->device));
  cudaStream_t st = (cudaStream_t)stream;
  TRY(setup_shot(M, sh, false, st));
  const size_t ns = (size_t)sh->nt * sh->nrec;
  const bool dev = ns == 0 || is_device_ptr(seis);
  float* sd = seis;
  if (!dev) {
    TRY(ensure_stage(M, ns));
    sd = M->stage;
  }
  // The whole shot is one CUDA graph (captured once per receiver geometry, output buffer and
  // step count, replayed afterwards), so small grids and thin slabs are not launch-bound.  With
  // an NCCL communicator the graph holds the halo send/recv groups (on the side stream of the
  // overlapped exchange) and the seismogram all-reduce: every rank captures the same sequence
  // of NCCL calls.  Peer halos (stream memory-operation flags) and every-launch profiling run
  // eagerly; graph-sampled profiling (seis_profile(S > 1)) keeps the graph.
  const bool use_graph = (!prof::on || prof::sample > 1) && !M->peer && !getenv("SEIS_NO_GRAPH");
  const int pmode = prof::on ? prof::sample : 0;
  const int pkey[2] = {pmode, pmode > 1 ? prof::epoch : 0};
  if (persist_ok(M)) {
    TRY(forward_persist(M, sh, sd, ns, st));
  } else if (use_graph) {
    uint64_t key = fnv1a(&sd, sizeof(sd), M->shot_key);  // (the wavelet is read on the device)
    key = fnv1a(&sh->nt, sizeof(int32_t), key);
    key = fnv1a(pkey, sizeof(pkey), key);  // (a graph with or without profiling event nodes)
    if (!M->gexec || M->gkey != key) {
      if (M->gexec) {
        cudaGraphExecDestroy(M->gexec);
        M->gexec = nullptr;
      }
      if (!M->cap) CK(cudaStreamCreateWithFlags(&M->cap, cudaStreamNonBlocking));
      CK(cudaStreamSynchronize(st));
      for (int k = 0; k < prof::NK; ++k) prof::glo[k] = prof::used[k];
      CK(cudaStreamBeginCapture(M->cap, cudaStreamCaptureModeThreadLocal));
      seis_status rc = forward_loop(M, sh, sd, ns, M->cap);
      for (int k = 0; k < prof::NK; ++k) prof::ghi[k] = prof::used[k];
      cudaGraph_t graph = nullptr;
      cudaError_t e = cudaStreamEndCapture(M->cap, &graph);
      if (rc != SEIS_OK) {
        if (graph) cudaGraphDestroy(graph);
        return rc;
      }
      if (e != cudaSuccess) return fail(SEIS_ECUDA, "graph capture: %s", cudaGetErrorString(e));
      e = cudaGraphInstantiate(&M->gexec, graph, 0);
      cudaGraphDestroy(graph);
      if (e != cudaSuccess) {
        M->gexec = nullptr;
        return fail(SEIS_ECUDA, "graph instantiate: %s", cudaGetErrorString(e));
      }
      M->gkey = key;
      M->g_launches = g_launches;
      M->gcur.clear();  // the host bookkeeping the capture ran (final level of every slab)
      for (Slab& S : M->slabs) M->gcur.push_back(S.cur);
    }
    CK(cudaGraphLaunch(M->gexec, st));
    g_launches = M->g_launches;
    for (size_t s = 0; s < M->slabs.size(); ++s) M->slabs[s].cur = M->gcur[s];
  } else {
    TRY(forward_loop(M, sh, sd, ns, st));
  }
  if (!dev && ns) CK(cudaMemcpyAsync(seis, sd, ns * sizeof(float), cudaMemcpyDeviceToHost, st));
  CK(cudaStreamSynchronize(st));
  if (use_graph && pmode > 1) CK(prof::harvest());  // (this replay's event nodes are complete)
  M->last_nt = sh->nt;
  return SEIS_OK;
}

seis_status seis_migrate(seis_model* M, const seis_shot* sh, const float* data, float* image,
                         void* stream) {
  g_launches = 0;
  if (!M) return fail(SEIS_EINVAL, "null model");
  if (!sh) return fail(SEIS_EINVAL, "null shot");
  if (!image) return fail(SEIS_EINVAL, "null image");
  if (sh->nrec > 0 && !data) return fail(SEIS_EINVAL, "null data");
  if (sh->snap_period < 1) return fail(SEIS_EINVAL, "snap_period must be >= 1");
  CK(cudaSetDevice(M->device));
  cudaStream_t st = (cudaStream_t)stream;
  const seis_grid& g = M->g;
  const int nt = sh->nt, snap = sh->snap_period;
  TRY(setup_shot(M, sh, false, st));
  // snapshot pool (O14): nsnap fields of the process slab, or (checkpointing, f2) the last
  // segment's c snapshots + nckpt source-state checkpoints
  const int nsnap = nt >= 1 ? (nt - 1) / snap : 0;
  const int c = sh->ckpt_period > 0 ? std::min(sh->ckpt_period, std::max(nsnap, 1)) : std::max(nsnap, 1);
  const int nseg = nsnap > 0 ? (nsnap + c - 1) / c : 0;
  const int nckpt = nseg > 1 ? nseg - 1 : 0;
  const size_t slab_pts = (size_t)M->pnzl * g.ny * g.nx;
  const size_t st_elems = nckpt ? state_elems(M) : 0;
  if (sh->snap_bits != 0 && sh->snap_bits != 32 && sh->snap_bits != 24)
    return fail(SEIS_EINVAL, "snap_bits must be 0, 32 or 24");
  const bool s24 = sh->snap_bits == 24;
  const size_t esz = s24 ? 3 : 4;  // bytes per snapshot value
  // (pool floats of the snapshot region, 256-byte aligned so the checkpoints stay aligned)
  const size_t snap_elems = ((size_t)std::min(c, nsnap) * slab_pts * esz + 255) / 256 * 64;
  const size_t need = snap_elems + (size_t)nckpt * st_elems;
  if (need > M->pool_elems) {
    size_t freeb = 0, totb = 0;
    cudaMemGetInfo(&freeb, &totb);
    if (M->pool) {
      cudaFree(M->pool);
      M->allocs.erase(std::find(M->allocs.begin(), M->allocs.end(), (void*)M->pool));
      M->pool = nullptr;
      M->pool_elems = 0;
    }
    void* p = nullptr;
    cudaError_t e = cudaMalloc(&p, need * sizeof(float));
    if (e != cudaSuccess) {
      cudaGetLastError();
      return fail(SEIS_ENOMEM, "snapshot pool needs %zu bytes (%d snapshots, %d checkpoints), %zu free",
                  need * 4, std::min(c, nsnap), nckpt, freeb);
    }
    M->allocs.push_back(p);
    M->pool = (float*)p;
    M->pool_elems = need;
  }
  float* ckpt0 = M->pool + snap_elems;  // checkpoint slot q = state at level (q + 1) c snap
  auto slot_of = [&](int q) { return ckpt0 + (size_t)q * st_elems; };
  std::vector<int> ckpt_cur(nckpt, 0);  // ISO: which buffer holds u^n at the checkpoint
  // pool pointers of snapshot index i (j = (i + 1) snap), which lives in segment i / c
  // snapshot i: fp32 [slab_pts] per snapshot, or (24-bit) a uint16 plane [slab_pts] followed by
  // a uint8 plane [slab_pts]; each slab's part starts at its z offset within the plane(s)
  auto snap_ptrs = [&](int i, std::vector<float*>& v) {
    const size_t off = (size_t)(i % c) * slab_pts;
    for (size_t s = 0; s < M->slabs.size(); ++s)
      v[s] = (float*)((char*)M->pool + (off + (size_t)(M->slabs[s].d.z0 - M->pz0) * g.ny * g.nx) * (s24 ? 2 : 4));
  };
  auto lo_plane = [&](int i, size_t s) {  // 24-bit: the uint8 plane of slab s of snapshot i
    return (uint8_t*)M->pool + (size_t)c * slab_pts * 2 + (size_t)(i % c) * slab_pts +
           (size_t)(M->slabs[s].d.z0 - M->pz0) * g.ny * g.nx;
  };
  const size_t nsl = M->slabs.size();
  // store snapshot i (level (i + 1) snap) of the current state in the 24-bit format
  auto snap24 = [&](int i) -> seis_status {
    std::vector<float*> dst(nsl);
    snap_ptrs(i, dst);
    for (size_t s = 0; s < nsl; ++s) {
      Slab& S = M->slabs[s];
      const float* f0 = M->kind == SEIS_ELASTIC ? S.fld[ESXX] : out_field(M, S, 0);
      const float* f1 = M->kind == SEIS_ELASTIC ? S.fld[ESYY] : f0;
      const float* f2 = M->kind == SEIS_ELASTIC ? S.fld[ESZZ] : f0;
      const int nf = M->kind == SEIS_ELASTIC ? 3 : 1;
      snap24_kernel<<<8 * 148, 256, 0, st>>>((uint16_t*)dst[s], lo_plane(i, s), f0, f1, f2, nf, S.d);
      CKL();
    }
    return SEIS_OK;
  };
  // image / data staging
  const bool img_dev = is_device_ptr(image);
  const size_t nd = (size_t)nt * sh->nrec;
  const bool data_dev = nd == 0 || is_device_ptr(data);
  float* img_d = image;
  const float* data_d = data;
  TRY(ensure_stage(M, (img_dev ? 0 : slab_pts) + (data_dev ? 0 : nd)));
  if (!img_dev) {
    img_d = M->stage;
    CK(cudaMemcpyAsync(img_d, image, slab_pts * sizeof(float), cudaMemcpyHostToDevice, st));
  }
  if (!data_dev) {
    float* dd = M->stage + (img_dev ? 0 : slab_pts);
    CK(cudaMemcpyAsync(dd, data, nd * sizeof(float), cudaMemcpyHostToDevice, st));
    data_d = dd;
  }
  // Forward source propagation over steps [n0, n1), storing the snapshots of segment `seg`
  // (all segments when seg < 0 and there is no checkpointing) and, in the first pass,
  // the checkpoints at the segment starts.
  std::vector<float*> snapp(M->slabs.size());
  auto forward = [&](int n0, int n1, int seg, bool first) -> seis_status {
    for (int n = n0; n < n1; ++n) {
      if (first && nckpt && n > 0 && n % (c * snap) == 0 && n / (c * snap) <= nckpt) {
        const int q = n / (c * snap) - 1;
        TRY(state_copy(M, slot_of(q), true, st));
        ckpt_cur[q] = M->slabs[0].cur;
      }
      const int j = n + 1;
      bool take = (j % snap == 0) && j <= nt - 1;
      if (take && (j / snap - 1) / c != seg) take = false;
      if (take && !s24) snap_ptrs(j / snap - 1, snapp);
      TRY(step(M, n, true, take && !s24 ? &snapp : nullptr, nullptr, nullptr, st));
      if (take && s24) TRY(snap24(j / snap - 1));
    }
    return SEIS_OK;
  };
  // ---- forward phase: source wavefield, snapshots S_j of the last segment (all of them
  // without checkpointing), checkpoints at the starts of the other segments
  TRY(zero_state(M, st));
  TRY(forward(0, nt, nseg - 1, true));
  // ---- backward phase: receiver wavefield from zero, same operator
  TRY(setup_shot(M, sh, true, st));
  TRY(zero_state(M, st));
  std::vector<SnapRef> Sp(M->slabs.size());
  std::vector<float*> Ip(M->slabs.size()), tmp(M->slabs.size());
  for (size_t s = 0; s < M->slabs.size(); ++s)
    Ip[s] = img_d + (size_t)(M->slabs[s].d.z0 - M->pz0) * g.ny * g.nx;
  int loaded = nseg - 1;  // segment whose snapshots are in the pool
  for (int m = 0; m < nt; ++m) {
    // imaging of level j = nt - m (the INPUT of this step, R^m) fused into the step kernel
    const int j = nt - m;
    const bool im = (j % snap == 0) && j >= snap && j <= nt - 1;
    if (im) {
      const int i = j / snap - 1, seg = i / c;
      if (seg != loaded) {
        // recompute segment seg from its checkpoint (zero state for seg 0).  The receiver
        // state is parked in checkpoint slot seg (the slot of segment seg + 1, consumed or
        // unused by now) and restored afterwards.
        const int rcur = M->slabs[0].cur;
        TRY(state_copy(M, slot_of(seg), true, st));
        if (seg == 0) {
          TRY(zero_state(M, st));
        } else {
          for (Slab& S : M->slabs) S.cur = ckpt_cur[seg - 1];
          TRY(state_copy(M, slot_of(seg - 1), false, st));
        }
        const int last_j = std::min((seg + 1) * c, nsnap) * snap;
        TRY(forward(seg * c * snap, last_j, seg, false));
        for (Slab& S : M->slabs) S.cur = rcur;
        TRY(state_copy(M, slot_of(seg), false, st));
        loaded = seg;
      }
      snap_ptrs(i, tmp);
      for (size_t s = 0; s < M->slabs.size(); ++s) {
        Sp[s] = SnapRef{};
        if (s24) {
          Sp[s].h16 = (const uint16_t*)tmp[s];
          Sp[s].l8 = lo_plane(i, s);
        } else {
          Sp[s].s32 = tmp[s];
        }
      }
    }
    // step + receiver injection of data[nt-1-m] (all receivers, one launch per slab)
    TRY(step(M, m, false, nullptr, im ? &Sp : nullptr, im ? &Ip : nullptr, st,
             sh->nrec ? data_d + (size_t)(nt - 1 - m) * sh->nrec : nullptr));
  }
  if (!img_dev) CK(cudaMemcpyAsync(image, img_d, slab_pts * sizeof(float), cudaMemcpyDeviceToHost, st));
  CK(cudaStreamSynchronize(st));
  M->last_nt = nt;
  return SEIS_OK;
}

seis_status seis_get_field(const seis_model* Mc, int32_t which, float* dst, void* stream) {
  seis_model* M = const_cast<seis_model*>(Mc);
  if (!M || !dst) return fail(SEIS_EINVAL, "null argument");
  const int nf = nfields(M->kind);
  if (which < 0 || which >= nf) return fail(SEIS_EINVAL, "field index %d out of range", which);
  CK(cudaSetDevice(M->device));
  cudaStream_t st = (cudaStream_t)stream;
  const seis_grid& g = M->g;
  const size_t slab_pts = (size_t)M->pnzl * g.ny * g.nx;
  const bool dev = is_device_ptr(dst);
  float* out = dst;
  if (!dev) {
    TRY(ensure_stage(M, slab_pts));
    out = M->stage;
  }
  for (Slab& S : M->slabs) {
    int f = which;
    if (M->kind == SEIS_ISO) f = which == 0 ? S.cur : 1 - S.cur;
    unpad_kernel<<<1024, 256, 0, st>>>(out + (size_t)(S.d.z0 - M->pz0) * g.ny * g.nx, S.fld[f], S.d);
    CKL();
  }
  if (!dev) CK(cudaMemcpyAsync(dst, out, slab_pts * sizeof(float), cudaMemcpyDeviceToHost, st));
  CK(cudaStreamSynchronize(st));
  return SEIS_OK;
}

}  // extern "C"
