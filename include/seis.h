/*
 * seis.h — C ABI of the B200-native seismic modeling / RTM hot path.
 *
 * Paper: Qawasmeh, Chapman, Hugues, Calandra, "GPU Technology Applied to
 * Reverse Time Migration and Seismic Modeling via OpenACC", PMAM'15 (PPoPP'15
 * workshop).  "P:<line>" cites /root/reference/PAPER.md; readings of passages
 * the paper leaves open are DESIGN.md §3 O1..O19.
 *
 * What the library computes (one call = one shot, Algorithm 1):
 *   seis_forward_model  seismic modeling (forward phase): time-stepped 8th-order
 *                       finite differences for Eq 1 (ISO), Eq 2
 *                       (ACOUSTIC, variable density) or Eq 3 (ELASTIC
 *                       velocity-stress), absorbing layers,
 *                       source injection each step and receiver sampling
 *                       ("predicts the seismograms").
 *   seis_migrate        reverse-time migration (Alg 1): forward
 *                       source propagation with snapshots kept in HBM (P:177,
 *                       O14), backward receiver propagation with the same
 *                       operator and all receivers injected in one launch
 *                       per step, zero-lag cross-correlation imaging
 *                       I += S * R (O15) accumulated over calls (sum_s).
 *
 * Conventions (all functions):
 *   - extern "C", never throw, return seis_status; seis_last_error() gives a
 *     thread-local message for the last non-OK status on this thread.
 *   - Arrays are C order [z][y][x] (x fastest), z = depth, k = 0 = top.
 *   - Single precision (fp32) storage and arithmetic ("All computations
 *     were carried out in single precision").
 *   - Buffers marked "host or device" may be either: the library inspects the
 *     pointer (cudaPointerGetAttributes) and stages host memory through device
 *     buffers itself.
 *   - Calls that take a stream are synchronous with respect to that stream on
 *     return (so CUDA / NCCL errors are reported by status).  stream = NULL
 *     means the legacy default stream.
 *   - The product path has no CPU fallback: without a CUDA device every
 *     compute call fails with SEIS_ECUDA.
 */
#ifndef SEIS_H
#define SEIS_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
  SEIS_OK = 0,
  SEIS_EINVAL = 1,       /* bad argument: null pointer, out-of-grid position, nt < 1, ... */
  SEIS_ECFL = 2,         /* Courant bound violated (O5) */
  SEIS_ENOMEM = 3,       /* device allocation failed or snapshot pool over budget */
  SEIS_ECUDA = 4,        /* CUDA runtime error (incl. "no device") */
  SEIS_ENCCL = 5,        /* NCCL error */
  SEIS_EUNSUPPORTED = 6  /* valid request this version does not implement */
} seis_status;

typedef enum {
  SEIS_ISO = 0,       /* Eq 1: constant-density isotropic, 2nd order in time, 25-point Laplacian */
  SEIS_ACOUSTIC = 1,  /* Eq 2: variable-density acoustic, staggered first-order (p, q) */
  SEIS_ELASTIC = 2    /* Eq 3: isotropic elastic velocity-stress, staggered (v, sigma) */
} seis_kind;

typedef struct seis_model seis_model; /* opaque; owns every device allocation of a model */
typedef struct seis_comm seis_comm;   /* opaque; an NCCL communicator + its stream */

/* Grid / physics description ("operators with a 3D stencil width of 8"). */
typedef struct {
  int32_t nx, ny, nz;   /* GLOBAL grid points; each >= 1 */
  float h;              /* uniform spacing dx = dy = dz (m), > 0 (O1) */
  float dt;             /* time step (s), > 0; must satisfy the Courant bound (O5) */
  int32_t nb;           /* absorbing-layer width in points, inside the grid; 0 = zero-Dirichlet
                           walls.  ISO: damped-wave layer (O6); ACOUSTIC/ELASTIC: C-PML (O7).
                           Must satisfy 3*nb <= min(nx, ny, nz). */
  int32_t free_surface; /* ELASTIC only: 1 = traction-free top (O16), no layer on the top face */
  float pml_R;          /* target reflection coefficient, 0 < R < 1 (default 1e-3) */
  float pml_f;          /* C-PML alpha reference frequency (Hz), >= 0 (default: source peak) */
  int32_t slabs;        /* z-slabs per PROCESS (>= 1).  > 1 runs the z-slab domain
                           decomposition on one GPU with direct ghost-plane stores
                           (f4); results are bitwise identical for every value. */
  int32_t iso_pml;      /* ISO absorbing layer ("standard PML ... in our second order
                           (isotropic) formulation"): 0 = damped wave (O6, default), 1 =
                           split-field PML (O6b: u = u^(x) + u^(y) + u^(z) inside the layers,
                           (d_t + eta_d)^2 u^(d) = v^2 d_d^2 u).  Must be 0 for other kinds
                           (EUNSUPPORTED). */
} seis_grid;

/* One shot ("one shot profile"). All arrays are borrowed for the call only. */
typedef struct {
  int32_t sx, sy, sz;        /* source node (global indices) */
  const float* wavelet;      /* HOST [nt]: injected samples s[n] (O11): ISO w(n dt);
                                ACOUSTIC / ELASTIC G((n+1/2) dt), G = integral of w */
  int32_t nt;                /* time steps, >= 1 */
  int32_t nrec;              /* receivers, >= 0 */
  const int32_t* rec;        /* HOST [nrec][3] = (x, y, z) global nodes (O12); duplicates allowed */
  int32_t rec_component;     /* ELASTIC: 0 vx, 1 vy, 2 vz, 3 pressure -(sxx+syy+szz)/3 (O13);
                                ignored for ISO (records u) and ACOUSTIC (records p) */
  int32_t snap_period;       /* >= 1: snapshot + imaging cadence (RTM only, O14) */
  int32_t ckpt_period;       /* RTM source-wavefield storage ("simulates the source
                                wave-field in both the forward and backward phases"):
                                0  = every snapshot S_j kept in the HBM pool (O14);
                                c >= 1 = checkpointing: snapshots are grouped in segments of c; the
                                forward phase keeps only the full source state (fields incl. ghost
                                planes + C-PML memory) at the start of segments 1.., and the last
                                segment's snapshots; the backward phase recomputes each earlier
                                segment's snapshots from its checkpoint just before they are imaged
                                (one extra forward pass at most).  Results are bitwise identical to
                                c = 0 (same kernels, same order of operations). */
  int32_t snap_bits;         /* RTM snapshot storage precision (SURVEY §8f f2's compressed-snapshot
                                alternative): 0 or 32 = fp32 (default); 24 = every snapshot value
                                rounded to nearest-even to 24 bits of its fp32 pattern (sign, 8-bit
                                exponent, 15 mantissa bits: relative rounding <= 2^-16), stored as
                                a 16-bit and an 8-bit plane: 3/4 of the fp32 pool.  No scale: the
                                stored value depends on the fp32 value only, so images stay bitwise
                                invariant under the z-slab decomposition and checkpointing; they
                                differ from the fp32-snapshot image by the rounding, ~1e-5
                                relative (inside the 1e-3 image bar).  EINVAL for other values. */
} seis_shot;

/* ---- multi-GPU (one process per GPU; z-slab decomposition, §8e) ---- */
/* Writes a fresh NCCL unique id (128 bytes) to broadcast to all ranks. */
seis_status seis_comm_unique_id(uint8_t id[128]);
/* Creates the communicator of `rank` among `nranks` on CUDA device `device`.
 * Collective over all ranks.  *out is owned by the caller (seis_comm_destroy). */
seis_status seis_comm_create(int32_t nranks, int32_t rank, const uint8_t id[128], int32_t device,
                             seis_comm** out);
seis_status seis_comm_destroy(seis_comm* comm);
/* Shot-parallel RTM (sum over shots of P:111 across ranks): every rank
 * migrates its own shots on a full-grid replica (comm = NULL model) into a local image,
 * then this all-reduces (sums) the n floats of `image` (device) over the communicator in
 * place.  Collective; synchronous w.r.t. `stream` on return. */
seis_status seis_image_reduce(seis_comm* comm, float* image, uint64_t n, void* stream);

/* ---- model ---- */
/* Creates a model: validates the grid (EINVAL), the Courant bound (ECFL), the
 * kind's requirements (ELASTIC needs vs; free_surface needs ELASTIC: EUNSUPPORTED),
 * uploads this process's z-slab and precomputes per-point coefficients (O1..O9).
 *   vp  HOST [nz_local][ny][nx] P velocity (m/s) of this process's slab
 *       (the whole grid when comm == NULL; slab bounds from seis_model_slab /
 *       seis_slab_bounds); every value > 0
 *   vs  HOST, same shape: S velocity (m/s), 0 <= vs <= vp/sqrt(2) (lambda >= 0);
 *       ELASTIC only (else NULL)
 *   rho HOST, same shape: density (kg/m^3) > 0; ACOUSTIC and ELASTIC (else NULL)
 * The arrays are only read during the call.  comm = NULL: single process.
 * device: CUDA device ordinal the model lives on. */
seis_status seis_model_create(const seis_grid* grid, seis_kind kind, const float* vp,
                              const float* vs, const float* rho, seis_comm* comm, int32_t device,
                              seis_model** out);
/* z-slab of `rank` among `nranks` for a grid of nz points (pure arithmetic, no device). */
seis_status seis_slab_bounds(int32_t nz, int32_t nranks, int32_t rank, int32_t* z0,
                             int32_t* nz_local);
/* This process's slab [z0, z0 + nz_local) of the global grid. */
seis_status seis_model_slab(const seis_model* model, int32_t* z0, int32_t* nz_local);
seis_status seis_model_destroy(seis_model* model);

/* ---- direct ghost-plane stores between ranks ----
 * The "sub-domains" of P:175 exchange their 4 boundary z-planes every half step.  By
 * default the ranks do that with NCCL send/recv overlapped with the interior updates.  In
 * peer mode the kernel that produces an exchanged field stores its first / last 4 planes
 * straight into the neighbouring rank's ghost planes (NVLink peer stores through CUDA IPC
 * mappings); the ranks order those stores with 32-bit flag words written and waited on by
 * stream memory operations.  No NCCL call is left in the time step.
 *
 * Peer-only communicator: no NCCL at all (e.g. two ranks sharing one GPU, which NCCL
 * rejects).  vmax = the maximum vp over the WHOLE grid, reduced by the caller (the absorbing
 * profiles and the Courant check need the global value; an NCCL communicator reduces it
 * itself).  With a peer-only communicator seis_forward_model does NOT all-reduce the
 * seismogram: each rank's `seis` holds the columns of the receivers its slab owns and zeros
 * elsewhere, and the caller sums them (exact: one owner per column).  EINVAL on bad args. */
seis_status seis_comm_create_peer(int32_t nranks, int32_t rank, int32_t device, double vmax,
                                  seis_comm** out);
/* Step 1 of peer mode, on every rank after seis_model_create (model with a communicator,
 * nranks >= 2, grid.slabs == 1): writes this rank's blob -- CUDA IPC handles of its state
 * fields, coefficient arrays and flag words -- to `blob` (host, capacity `cap` bytes) and its
 * size to *len.  blob = NULL: size query only.  EINVAL: not a multi-rank model, cap too small;
 * EUNSUPPORTED: SEIS_AC_FUSED=1 (the fused step exchanges 8 planes of p). */
seis_status seis_model_peer_export(seis_model* model, uint8_t* blob, uint64_t cap, uint64_t* len);
/* Step 2, after every rank has exported and the blobs were exchanged by the caller (any
 * transport, e.g. torch.distributed all_gather_object): maps the blobs of rank-1 (lo_blob,
 * the slab above; NULL on rank 0) and rank+1 (hi_blob, the slab below; NULL on the last
 * rank), fills the coefficient ghost planes from them and switches the model to peer mode
 * for the rest of its life.  Blobs are only read during the call.  EINVAL: a needed blob is
 * missing / short / from another decomposition, or export did not run; ECUDA: mapping failed.
 * Subsequent forward_model / migrate calls are collective over the neighbouring ranks (every
 * whole-state reset is fenced by a flag barrier). */
seis_status seis_model_peer_import(seis_model* model, const uint8_t* lo_blob, uint64_t lo_len,
                                   const uint8_t* hi_blob, uint64_t hi_len);

/* ---- the hot path ---- */
/* Seismic modeling of one shot from a zero state (Alg 1 forward phase).
 *   seis  host or device [nt][nrec] fp32, written in full: seis[n][r] = field^{n+1}(x_r) (O13).
 *         With an NCCL communicator every rank receives the full array (NCCL all-reduce of
 *         the rank-owned entries; exact because exactly one rank owns each receiver); with a
 *         peer-only communicator (seis_comm_create_peer) each rank's array holds its own
 *         receivers' columns and zeros elsewhere (the caller sums them).
 * With peer halos (seis_model_peer_import) the call is collective over the neighbouring
 * ranks, like every call that steps the wavefield. */
seis_status seis_forward_model(seis_model* model, const seis_shot* shot, float* seis,
                               void* stream);
/* Reverse-time migration of one shot.  ISO images u, ACOUSTIC p, ELASTIC the pressure
 * -(sxx+syy+szz)/3 (receivers inject like the explosive source).
 *   data  host or device [nt][nrec] fp32 observed data (replicated on every rank)
 *   image host or device [nz_local][ny][nx] fp32, ACCUMULATED (+=), never zeroed
 * Snapshot pool: nsnap = (nt-1)/snap_period fields of nz_local*ny*nx floats in HBM
 * (ckpt_period = 0), or min(c, nsnap) snapshot fields + (ceil(nsnap/c) - 1) source-state
 * checkpoints (ckpt_period = c); SEIS_ENOMEM (with the byte count in seis_last_error) if
 * it does not fit. */
seis_status seis_migrate(seis_model* model, const seis_shot* shot, const float* data,
                         float* image, void* stream);

/* ---- inspection (tests) ---- */
/* Copies the final state field `which` of the last call (local slab, compact
 * [nz_local][ny][nx]) to dst (host or device).
 *   ISO: 0 = u^{nt}, 1 = u^{nt-1}.  ACOUSTIC: 0 = p, 1 = qx, 2 = qy, 3 = qz.
 *   ELASTIC: 0..8 = vx, vy, vz, sxx, syy, szz, sxy, sxz, syz. */
seis_status seis_get_field(const seis_model* model, int32_t which, float* dst, void* stream);
/* Device bytes a model + one migrate call needs per process (state, coefficients,
 * C-PML slabs, ISO split-field PML components, snapshot pool: 4 or, with snap_bits = 24, 3 bytes
 * per snapshot value, and the checkpoints of ckpt_period). shot may be NULL (modeling only). */
seis_status seis_memory_required(const seis_grid* grid, seis_kind kind, const seis_shot* shot,
                                 int32_t nranks, uint64_t* bytes);
/* Per-kernel CUDA-event timing (profiling / bench.py).  seis_profile(1) resets the
 * counters and starts recording an event pair on the launching stream around every
 * launch (launches then run eagerly, no shot graph); seis_profile(S), S > 1, resets and
 * keeps the forward shot's CUDA graph, with event-record nodes around the launches of
 * every S-th time step inside it, read back after each replay (the measured path is the
 * production one; calling seis_profile(S) again in that mode only zeroes the counters, the
 * graph is kept); seis_profile(0) stops.  seis_profile_read synchronises on the recorded
 * events and returns the summed device time and launch count (sampled launches in the
 * graph-sampled mode) of kernel id
 *   0 iso_step  1 ac_v  2 ac_p  3 el_v  4 el_s  5 inject  6 gather
 *   7 halo exchange (copies / NCCL)  8 free-surface mirror  9 fused acoustic step
 *   10 ISO 2-step kernel.
 * Process-wide, not thread-safe; meant for single-threaded measurement runs. */
seis_status seis_profile(int32_t enable);
seis_status seis_profile_read(int32_t kernel, double* total_ms, int64_t* launches);
/* Number of kernel launches issued by the last forward_model / migrate call on this thread. */
int64_t seis_last_launch_count(void);
/* Library version string. */
const char* seis_version(void);
/* Thread-local message of the last non-OK status; valid until the next call on this thread. */
const char* seis_last_error(void);

#ifdef __cplusplus
}
#endif
#endif /* SEIS_H */
