// kernels_acoustic_step.cuh — one full acoustic time step (Eq 2: V then P, O2/O8)
// in ONE persistent launch, without halo recomputation or double-buffered state (SURVEY §8f f1:
// "single-pass fused staggered kernels", 56 -> 40 B per point and step).
//
// The split pair (kernels_acoustic.cuh) moves 56 B per point: V reads p, q, rho and writes q
// (32 B), P reads q, p, K and writes p (24 B).  One sweep that reads p^n, q^{n-1/2}, rho, K
// once and writes q^{n+1/2}, p^{n+1} once moves 40 B.  P at (x, y, k) needs q^{n+1/2} on the
// cross x-4..x+3, y-4..y+3, k-4..k+3, i.e. values produced by the neighbouring tiles.  Round 1
// recomputed those halos in every block (double-buffered state, +50 % V work on the y halo:
// slower than the split pair).  Here the tiles instead EXCHANGE them through L2 as a wavefront:
//
//   * one CTA per (128 x 14) xy tile, all tiles co-resident (cooperative launch; one CTA per SM),
//     each marching the whole z range: at iteration j it runs V at plane j and P at plane
//     j - L (L = 4), in place (q^{n+1/2} over q^{n-1/2}, p^{n+1} over p^n);
//   * P(k) needs q^{n+1/2}(k) from the x / y neighbour tiles: once every consumer warp of a
//     tile has arrived on the stage of V(k) (after its q stores), the producer thread publishes
//     the plane with a release add on the tile's counter; a producer acquires the own + 4
//     neighbour counters >= k + 1 before it TMA-loads the q_x (x halo) and q_y (y halo) tiles of
//     plane k for P -- they come from L2, written a few planes earlier;
//   * the in-place overwrite is safe: a tile's p^n(k) halo is read only by its neighbours' V(k),
//     which completes (TMA data consumed) before this tile's P(k) may start (the neighbours'
//     counters gate it); q^{n-1/2} is read only pointwise by its own V;
//   * p^n (needed 3 planes back, 4 ahead, and at plane j - 4 for P) stays in a per-thread
//     register queue along z, q_z^{n+1/2} (4 back, 3 ahead) in an 8-plane shared-memory ring
//     (each thread its own column); both are 8 deep because P(j - 4) runs before V(j).
//
// Warp roles: 32 x 14 consumer threads (4 x-points each) + 2 producer warps: one issues the
// V-stage TMA loads (ring NSV deep: p tile + halo 4, q_x, q_y, q_z, rho tile + 1, rho(k+1),
// p(k+4)) and publishes completed planes, the other the P-stage loads (ring NSP deep: q_x new +
// x halo, q_y new + y halo, dt K/h) once the counters allow.  Full / empty mbarriers per stage;
// no CTA-wide barrier in the march.
//
// Per-point arithmetic is the split kernels' expression for expression (same face buoyancy,
// same C-PML updates, same source add), so results are bitwise identical to the split pair
// (tested); DESIGN.md §6.
#pragma once
#include "common.cuh"
#include "kernels_acoustic.cuh"  // CpmlAxis

namespace seis {

// Tile: 128 x 14 points = 14 consumer warps (32 threads per row, 4 x-points each) + 2 producer
// warps = 16 warps, 4 per SM sub-partition, so each thread may hold 128 registers (the two
// z-queues alone take 64); a 512^2 plane is 4 x 37 = 148 tiles, one per SM of a B200
#ifndef SEIS_AS_TX
#define SEIS_AS_TX 128
#endif
#ifndef SEIS_AS_TY
#define SEIS_AS_TY 14
#endif
constexpr int AS_TX = SEIS_AS_TX;
constexpr int AS_TY = SEIS_AS_TY;
constexpr int AS_NTX = AS_TX / 4;            // consumer threads per row (4 x-points each)
constexpr int AS_CONS = AS_NTX * AS_TY;      // consumer threads
constexpr int AS_CWARPS = AS_CONS / 32;      // consumer warps (= counter increments per plane)
constexpr int AS_THREADS = AS_CONS + 64;     // + the two producer warps (V loads, P loads)
constexpr int AS_L = 4;                      // P lags V by L planes
#ifndef SEIS_AS_NSV
#define SEIS_AS_NSV 2
#endif
#ifndef SEIS_AS_NSP
#define SEIS_AS_NSP 3
#endif
constexpr int AS_NSV = SEIS_AS_NSV;

// L2 prefetch distance (planes) of the DRAM-sourced operands: the shared-memory rings are only
// NSV / NSP deep (one CTA per SM holds ~200 KB), so the HBM latency is covered by bringing each
// plane into L2 AS_PF planes before its TMA load (cp.async.bulk.prefetch.tensor, no smem)
#ifndef SEIS_AS_PF
#define SEIS_AS_PF 2
#endif
constexpr int AS_PF = SEIS_AS_PF;
// per-thread L2 prefetch of the C-PML slabs (prefetch.global.L2): measured slower (1.69 ms per
// 512^3 step with it, 1.50 without), off by default
#ifndef SEIS_AS_PSIPF
#define SEIS_AS_PSIPF 0
#endif
constexpr int AS_NSP = SEIS_AS_NSP;

struct AcSArgs {
  CUtensorMap mpt;             // p^n tile, box (64+8) x (TY+8), origin (i0-4, j0-4)
  CUtensorMap mqx, mqy, mqz;   // q^{n-1/2}, box 64 x TY (plane j)
  CUtensorMap mrt;             // rho tile, box (64+4) x (TY+1), origin (i0, j0)
  CUtensorMap mrz;             // rho, box 64 x TY (plane j+1)
  CUtensorMap mpq;             // p^n, box 64 x TY (plane j+4: z-queue feed)
  CUtensorMap mqxn;            // q_x^{n+1/2}, box (64+8) x TY, origin (i0-4, j0)  (P stage)
  CUtensorMap mqyn;            // q_y^{n+1/2}, box 64 x (TY+8), origin (i0, j0-4)  (P stage)
  CUtensorMap mk;              // dt K / h, box 64 x TY (L2 prefetch only)
  const float* __restrict__ p0;   // p (padded): warm-up loads of the z-queue
  float* p;                       // p^{n+1} stores (same array as p0)
  float* __restrict__ qx;
  float* __restrict__ qy;
  float* __restrict__ qz;
  const float* __restrict__ kk;   // dt K / h (padded): P's pointwise coefficient, by cp.async
  float dth;                      // dt / h
  int W, zlo;
  CpmlAxis cx, cy, cz;
  float* __restrict__ psx;        // psi_{p,x|y|z} (V)
  float* __restrict__ psy;
  float* __restrict__ psz;
  float* __restrict__ pqx;        // psi_{q,x|y|z} (P)
  float* __restrict__ pqy;
  float* __restrict__ pqz;
  Dims d;
  int ntx, nty;                   // tiles in x and y (gridDim.x = ntx * nty)
  unsigned* __restrict__ cnt;     // per-tile V progress counters (zeroed before the launch)
  long long src_o;
  SrcAmp src;
  float* __restrict__ snap;       // compact snapshot target (p^{n+1}), or nullptr
  SnapRef imgR;                   // imaging of the input level p^n, or nullptr (img)
  float* __restrict__ img;
  unsigned long long* trace;      // SEIS_AS_TRACE builds only: [tiles][nz][8] event times (ns)
};

// Event timeline of the fused step (tools/ac_step_trace.py; compiled in only with
// -DSEIS_AS_TRACE=1): per tile and plane, the global timer at 8 events.
#ifndef SEIS_AS_TRACE
#define SEIS_AS_TRACE 0
#endif
__device__ __forceinline__ unsigned long long gtimer() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
  return t;
}
#define AS_TRACE(k, ev)                                                                        \
  do {                                                                                         \
    if (SEIS_AS_TRACE && a.trace) a.trace[((size_t)tile * nz + (k)) * 48 + (ev)] = gtimer();  \
  } while (0)

struct AcSLayout {
  static constexpr int PW = AS_TX + 8, T = AS_TX * AS_TY, RW = AS_TX + 4;
  // V stage
  static constexpr int PT = 0, QX = PT + r32(PW * (AS_TY + 8)), QY = QX + r32(T), QZ = QY + r32(T),
                       R = QZ + r32(T), RZ = R + r32(RW * (AS_TY + 1)), PQ = RZ + r32(T), VSIZE = PQ + r32(T);
  static constexpr uint32_t VBYTES = (PW * (AS_TY + 8) + 5 * T + RW * (AS_TY + 1)) * 4;
  // P stage
  static constexpr int QXN = 0, QYN = QXN + r32(PW * AS_TY), PSIZE = QYN + r32(AS_TX * (AS_TY + 8));
  static constexpr uint32_t PBYTES = (PW * AS_TY + AS_TX * (AS_TY + 8)) * 4;
  // q_z^{n+1/2} ring: planes j-8 .. j-1 (8 slots; each thread reads and writes only its column)
  static constexpr int ZSIZE = 0;
  // C-PML memory variables in flight: per consumer thread and axis the 4 old values of the
  // next half step, brought by cp.async (no registers held while they travel)
  // (two sets: psi_p for V, psi_q for P; plus the 4 values of dt K/h for P)
  static constexpr int QSIZE = 7 * AS_CONS * 4;
  static constexpr size_t smem_bytes() {
    return ((size_t)AS_NSV * VSIZE + (size_t)AS_NSP * PSIZE + ZSIZE + QSIZE) * 4 + 128;
  }
};

// psi <- b psi + a dv; dv += psi (common.cuh psi_upd)
template <int NV>
__device__ __forceinline__ void psi_upd_s(float* dv, float* __restrict__ ps, const int* ix, const float* old,
                                          const float* ca, const float* cb) {
#pragma unroll
  for (int e = 0; e < NV; ++e)
    if (ix[e] >= 0) {
      const float v = fmaf(cb[e], old[e], ca[e] * dv[e]);
      ps[ix[e]] = v;
      dv[e] += v;
    }
}
// the same for a contiguous, 16-byte aligned group of 4 (one vector store)
__device__ __forceinline__ void psi_upd_v4(float* dv, float* __restrict__ ps, int base, const float* old,
                                           const float* ca, const float* cb) {
  F4 v;
#pragma unroll
  for (int e = 0; e < 4; ++e) {
    v.v[e] = fmaf(cb[e], old[e], ca[e] * dv[e]);
    dv[e] += v.v[e];
  }
  st4(ps + base, v);
}
template <bool SNAP, bool IMG>
__global__ void __launch_bounds__(AS_THREADS, 1) ac_step_kernel(const __grid_constant__ AcSArgs a) {
  using L = AcSLayout;
  constexpr int PW = L::PW, RW = L::RW;
  static_assert(L::QX % 32 == 0 && L::QY % 32 == 0 && L::R % 32 == 0 && L::RZ % 32 == 0 && L::PQ % 32 == 0 &&
                    L::VSIZE % 32 == 0 && L::QYN % 32 == 0 && L::PSIZE % 32 == 0,
                "128-byte tiles");
  extern __shared__ __align__(128) float sm_raw[];
  float* sm = align128(sm_raw);
  float* smv = sm;                          // AS_NSV V stages
  float* smp = sm + AS_NSV * L::VSIZE;      // AS_NSP P stages
  __shared__ __align__(8) uint64_t fullv[AS_NSV], emptyv[AS_NSV], fullp[AS_NSP], emptyp[AS_NSP];
  __shared__ CpmlTile<AS_TX, AS_TY> cpt;  // x / y C-PML coefficients of this tile (a, b, ah, bh)
  const Dims& d = a.d;
  const int tid = threadIdx.x;
  const int tile = blockIdx.x;
  const int tix = tile % a.ntx, tiy = tile / a.ntx;
  const int i0 = tix * AS_TX, j0 = tiy * AS_TY;
  const int nz = d.nzl;
  const int niter = nz + AS_L;
  if (tid == 0) {
    for (int s = 0; s < AS_NSV; ++s) {
      mbar_init(&fullv[s], 1);
      mbar_init(&emptyv[s], AS_CWARPS);
    }
    for (int s = 0; s < AS_NSP; ++s) {
      mbar_init(&fullp[s], 1);
      mbar_init(&emptyp[s], AS_CWARPS);
    }
    mbar_fence_init();
  }
  cpml_tile_fill(cpt, a.cx, a.cy, i0, j0, d.nx, d.ny, a.W > 0, tid, AS_THREADS);
  __syncthreads();

  if (tid >= AS_CONS) {
    // ---------------------------------------------------------------- producer warps
    // Lane 0 of each: blocking waits are fine, each thread has a single job.
    const int pw = (tid - AS_CONS) >> 5, lane = tid & 31;
    const int x = i0 + G, y = j0 + G;
    if (pw == 0 && lane == 0) {
      // V stages: no dependency beyond a free slot.  The slot of plane j - NSV is free again when
      // all consumer warps arrived on it, i.e. after they completed V(j - NSV) INCLUDING its
      // global q stores (the arrive follows them): that is when this thread publishes the plane
      // to the neighbour tiles (release add on the tile's counter = planes whose V is complete).
      unsigned* const mycnt = a.cnt + tile;
      for (int j = 0; j < nz + AS_NSV; ++j) {
        const int s = j % AS_NSV;
        if (j >= AS_NSV) {
          mbar_wait_nap(&emptyv[s], ((j / AS_NSV) - 1) & 1);
          AS_TRACE(j - AS_NSV, 8);
          fence_proxy_async_global();
          AS_TRACE(j - AS_NSV, 9);
          red_release_gpu_add(mycnt, 1u);
          AS_TRACE(j - AS_NSV, 1);
        }
        if (j >= nz) continue;
        float* st = smv + s * L::VSIZE;
        const int z = j + GZ;
        mbar_expect_tx(&fullv[s], L::VBYTES);
        tma_load_3d(st + L::PT, &a.mpt, &fullv[s], i0, j0, z);
        tma_load_3d(st + L::QX, &a.mqx, &fullv[s], x, y, z);
        tma_load_3d(st + L::QY, &a.mqy, &fullv[s], x, y, z);
        tma_load_3d(st + L::QZ, &a.mqz, &fullv[s], x, y, z);
        tma_load_3d(st + L::R, &a.mrt, &fullv[s], x, y, z);
        tma_load_3d(st + L::RZ, &a.mrz, &fullv[s], x, y, z + 1);
        tma_load_3d(st + L::PQ, &a.mpq, &fullv[s], x, y, z + 4);
        AS_TRACE(j, 0);
        if (AS_PF > 0 && j + AS_PF < nz + 4) {
          const int zp = z + AS_PF;
          tma_prefetch_3d(&a.mpq, x, y, zp + 4);
          tma_prefetch_3d(&a.mqx, x, y, zp);
          tma_prefetch_3d(&a.mqy, x, y, zp);
          tma_prefetch_3d(&a.mqz, x, y, zp);
          tma_prefetch_3d(&a.mrz, x, y, zp + 1);
          tma_prefetch_3d(&a.mk, x, y, zp - AS_L);
        }
      }
    } else if (pw == 1 && lane == 0) {
      // P stages: a free slot, then V(k) complete in this tile and its x / y neighbours
      // (acquire loads of their counters), then the q_x (x halo), q_y (y halo) and K tiles.
      const unsigned* cs[5] = {a.cnt + tile, tix > 0 ? a.cnt + tile - 1 : nullptr,
                               tix + 1 < a.ntx ? a.cnt + tile + 1 : nullptr,
                               tiy > 0 ? a.cnt + tile - a.ntx : nullptr,
                               tiy + 1 < a.nty ? a.cnt + tile + a.ntx : nullptr};
      unsigned seen[5] = {0u, 0u, 0u, 0u, 0u};
      for (int k = 0; k < nz; ++k) {
        const int s = k % AS_NSP;
        if (k >= AS_NSP) mbar_wait_nap(&emptyp[s], ((k / AS_NSP) - 1) & 1);
        AS_TRACE(k, 10);
        const unsigned need = (unsigned)(k + 1);  // V(0 .. k) complete
        for (;;) {
          bool ok = true;
#pragma unroll
          for (int c = 0; c < 5; ++c)
            if (cs[c] && seen[c] < need) seen[c] = ld_relaxed_gpu(cs[c]);  // (all in flight at once)
#pragma unroll
          for (int c = 0; c < 5; ++c) ok = ok && (!cs[c] || seen[c] >= need);
          if (ok) break;
          __nanosleep(SEIS_AS_NAP);
        }
        AS_TRACE(k, 11);
        fence_acq_rel_gpu();         // acquire: the q stores released with the counters
        fence_proxy_async_global();  // ... ordered before the TMA (async proxy) reads
        float* st = smp + s * L::PSIZE;
        const int z = k + GZ;
        mbar_expect_tx(&fullp[s], L::PBYTES);
        tma_load_3d(st + L::QXN, &a.mqxn, &fullp[s], i0, y, z);
        tma_load_3d(st + L::QYN, &a.mqyn, &fullp[s], x, j0, z);
        AS_TRACE(k, 2);
      }
    }
    return;
  }

  // ------------------------------------------------------------------ consumer threads
  const int tx = tid % AS_NTX, ty = tid / AS_NTX;
  const int x0 = i0 + 4 * tx, jy = j0 + ty;
  const bool own = (x0 < d.nx) && (jy < d.ny);
  const long long PS = d.PS;
  const long long oc = (long long)(jy + G) * d.PX + (x0 + G);
  const int Wl = a.W;
  const bool lx = Wl > 0 && (x0 < Wl || x0 + 3 >= d.nx - Wl);
  const bool ly = Wl > 0 && CpmlIdx::in(jy, d.ny, Wl, true);
  const float dth = a.dth;
  const int lane = tid & 31;
  const int pt = ty * AS_TX + 4 * tx;

  // queues along z (P runs before V in an iteration, so both are 8 deep):
  //   r (registers): at the top of iteration j, r[0..7] = p^n(j-4 .. j+3); P(j-4) uses r[0];
  //     then r shifts and V(j) appends p^n(j+4) (TMA stage) as r[7];
  //   q_z^{n+1/2} (shared ring, slot = plane mod 8, own column only): P(j-4) reads planes
  //     j-8 .. j-1, then V(j) writes plane j into the slot of plane j-8
  F4 r[8];
#pragma unroll
  for (int t = 0; t < 8; ++t) r[t] = ldg4(a.p0 + (long long)(t - 4 + GZ) * PS + oc);
  F4 zq[8];  // q_z^{n+1/2}(j-8 .. j-1) at the top of iteration j
#pragma unroll
  for (int t = 0; t < 8; ++t) zq[t] = F4{{0.f, 0.f, 0.f, 0.f}};
  // (per-plane source test: src_hit measured slower here, 1.55 vs 1.50 ms, r02_src_store_ab.log)
  const long long srel0 = a.src_o - oc;
  // Per-thread operands of the next half step travel by cp.async into this thread's slots while
  // the current one computes (no registers held, latency hidden): the C-PML memory variables
  // (V: psi_p at plane j, issued at the top of iteration j; P: psi_q at plane j - 3, issued
  // after P(j - 4) consumed its slots) and, with psi_q, dt K/h of P's plane.  The slabs and K
  // are prefetched into L2 AS_PF planes ahead.  Axis flags: lx / ly per thread, the z layer per
  // plane.  Each iteration commits exactly two cp.async groups (V's, then P's), so the group of
  // a half step is complete once at most one younger group is pending.
  constexpr int QS = AS_CONS * 4;  // axis stride of the slots
  // (16-byte copies / stores of a group's 4 memory variables need 16-byte aligned rows)
  const bool vec4 = (d.nx & 3) == 0 && x0 + 3 < d.nx;
  float* const psq_v = smp + AS_NSP * L::PSIZE + L::ZSIZE + 4 * tid;  // [3 axes] V slots
  float* const psq_p = psq_v + 3 * QS;                                 // [3 axes] P slots
  float* const ksl = psq_v + 6 * QS;                                   // dt K/h of P's plane
  auto psi_issue = [&](float* const* arr, float* psq, int k) {
    const int gz = k + d.z0;
    const bool lzk = Wl > 0 && CpmlIdx::in(gz, d.nz, Wl, a.zlo);
    if (own && lx) {  // x slab: the layer points of the group only (a few lanes per warp)
      int ix[4];
      psi_idx_x<4>(ix, d, Wl, x0, jy, k);
#pragma unroll
      for (int e = 0; e < 4; ++e)
        if (ix[e] >= 0) cp_async4(psq + e, arr[0] + ix[e], true);
    }
    // y / z slabs: the group's 4 values are contiguous; one 16-byte copy when aligned
    if (own && ly) {
      const int b = (k * (2 * Wl) + CpmlIdx::slot(jy, d.ny, Wl)) * d.nx + x0;
      if (vec4) {
        cp_async16(psq + QS, arr[1] + b);
      } else {
#pragma unroll
        for (int e = 0; e < 4; ++e)
          if (x0 + e < d.nx) cp_async4(psq + QS + e, arr[1] + b + e, true);
      }
    }
    if (own && lzk) {
      const int b = (CpmlIdx::slot(gz, d.nz, Wl) * d.ny + jy) * d.nx + x0;
      if (vec4) {
        cp_async16(psq + 2 * QS, arr[2] + b);
      } else {
#pragma unroll
        for (int e = 0; e < 4; ++e)
          if (x0 + e < d.nx) cp_async4(psq + 2 * QS + e, arr[2] + b + e, true);
      }
    }
  };
  auto psi_prefetch = [&](float* const* arr, int k) {  // one lane per 128-byte line
    const int gz = k + d.z0;
    if (!own || k >= nz) return;
    if (lx && (tx & 7) == 0) {  // (a row's layer slots are within 2 W contiguous floats)
      const int b = (k * d.ny + jy) * (2 * Wl) + (x0 < Wl ? 0 : Wl);
      prefetch_l2(arr[0] + b);
      prefetch_l2(arr[0] + b + Wl - 1);
    }
    if ((tx & 7) != 0) return;
    if (ly) prefetch_l2(arr[1] + (k * (2 * Wl) + CpmlIdx::slot(jy, d.ny, Wl)) * d.nx + x0);
    if (Wl > 0 && CpmlIdx::in(gz, d.nz, Wl, a.zlo))
      prefetch_l2(arr[2] + (CpmlIdx::slot(gz, d.nz, Wl) * d.ny + jy) * d.nx + x0);
  };
  float* const psv[3] = {a.psx, a.psy, a.psz};
  float* const psp[3] = {a.pqx, a.pqy, a.pqz};

  // (the first P, k = 0, finds its operands in the group issued at the end of iteration 3)
  for (int j = 0; j < niter; ++j) {
    if (j < nz) psi_issue(psv, psq_v, j);  // V(j)'s psi_p (its slots were consumed by V(j - 1))
    cp_async_commit();
    if (j >= AS_L) {
      // ================================ P at plane k = j - L (ac_p, same arithmetic)
      const int k = j - AS_L;
      const int s = k % AS_NSP;
      const long long o = (long long)(k + GZ) * PS + oc;
      const int gz = k + d.z0;
      const bool lz = Wl > 0 && CpmlIdx::in(gz, d.nz, Wl, a.zlo);
      if (tid == 0) AS_TRACE(k, 6);
      mbar_wait(&fullp[s], (k / AS_NSP) & 1);
      if (tid == 0) AS_TRACE(k, 3);
      const float* st = smp + s * L::PSIZE;
      const float* cxp = st + L::QXN + ty * PW + 4 * tx + 4;          // q_x(x0, jy)
      const float* cyp = st + L::QYN + (ty + 4) * AS_TX + 4 * tx;     // q_y(x0, jy)
      float xv[12];
      {
        const F4 a0 = lds4(cxp - 4), a1 = lds4(cxp), a2 = lds4(cxp + 4);
#pragma unroll
        for (int e = 0; e < 4; ++e) {
          xv[e] = a0.v[e];
          xv[4 + e] = a1.v[e];
          xv[8 + e] = a2.v[e];
        }
      }
      F4 yr[8];  // q_y rows jy-4 .. jy+3
#pragma unroll
      for (int m = 0; m < 8; ++m) yr[m] = lds4(cyp + (m - 4) * AS_TX);
      __syncwarp();
      if (lane == 0) mbar_arrive(&emptyp[s]);  // (everything of the stage is in registers)
      float dx[4], dy[4], dz[4];
#pragma unroll
      for (int e = 0; e < 4; ++e) {
        float t = SEIS_D1 * (xv[4 + e] - xv[3 + e]);
        t = fmaf(SEIS_D2, xv[5 + e] - xv[2 + e], t);
        t = fmaf(SEIS_D3, xv[6 + e] - xv[1 + e], t);
        dx[e] = fmaf(SEIS_D4, xv[7 + e] - xv[0 + e], t);
        t = SEIS_D1 * (yr[4].v[e] - yr[3].v[e]);
        t = fmaf(SEIS_D2, yr[5].v[e] - yr[2].v[e], t);
        t = fmaf(SEIS_D3, yr[6].v[e] - yr[1].v[e], t);
        dy[e] = fmaf(SEIS_D4, yr[7].v[e] - yr[0].v[e], t);
      }
      {  // q_z(k-4 .. k+3) = zq[0 .. 7]
#pragma unroll
        for (int e = 0; e < 4; ++e) {
          float t = SEIS_D1 * (zq[4].v[e] - zq[3].v[e]);
          t = fmaf(SEIS_D2, zq[5].v[e] - zq[2].v[e], t);
          t = fmaf(SEIS_D3, zq[6].v[e] - zq[1].v[e], t);
          dz[e] = fmaf(SEIS_D4, zq[7].v[e] - zq[0].v[e], t);
        }
      }
      cp_async_wait<1>();  // this thread's psi_q + K slots (P's group; V(j)'s may be pending)
      const F4 kv = lds4(ksl);
      float* const psq = psq_p;
      if (own) {
        if (lx) {
          int ix[4];
          float ca[4], cb[4];
          psi_idx_x<4>(ix, d, Wl, x0, jy, k);
          const F4 ov = lds4(psq);
#pragma unroll
          for (int e = 0; e < 4; ++e) {
            ca[e] = cpt.x[0][4 * tx + e];
            cb[e] = cpt.x[1][4 * tx + e];
          }
          psi_upd_s<4>(dx, a.pqx, ix, ov.v, ca, cb);
        }
        if (ly) {
          int iy[4];
          psi_idx_row<4>(iy, (k * (2 * Wl) + CpmlIdx::slot(jy, d.ny, Wl)) * d.nx + x0, x0, d.nx);
          const F4 ov = lds4(psq + QS);
          const float ya = cpt.y[0][ty], yb = cpt.y[1][ty];
          const float ca[4] = {ya, ya, ya, ya}, cb[4] = {yb, yb, yb, yb};
          if (vec4) psi_upd_v4(dy, a.pqy, iy[0], ov.v, ca, cb);
          else psi_upd_s<4>(dy, a.pqy, iy, ov.v, ca, cb);
        }
        if (lz) {
          int iz[4];
          psi_idx_row<4>(iz, (CpmlIdx::slot(gz, d.nz, Wl) * d.ny + jy) * d.nx + x0, x0, d.nx);
          const F4 ov = lds4(psq + 2 * QS);
          const float za = __ldg(a.cz.a + gz), zb = __ldg(a.cz.b + gz);
          const float ca[4] = {za, za, za, za}, cb[4] = {zb, zb, zb, zb};
          if (vec4) psi_upd_v4(dz, a.pqz, iz[0], ov.v, ca, cb);
          else psi_upd_s<4>(dz, a.pqz, iz, ov.v, ca, cb);
        }
        const F4 pv = r[0];  // p^n(k)
        F4 out;
#pragma unroll
        for (int e = 0; e < 4; ++e) out.v[e] = fmaf(kv.v[e], (dx[e] + dy[e]) + dz[e], pv.v[e]);
        const long long rel = srel0 - (long long)(k + GZ) * PS;
        if (rel >= 0 && rel < 4) {
#pragma unroll
          for (int e = 0; e < 4; ++e)
            if (rel == e) out.v[e] += a.src.get();
        }
        st4_masked(a.p + o, out, x0, d.nx, true);
        if (SNAP) st4_masked(a.snap + ((long long)k * d.ny + jy) * d.nx + x0, out, x0, d.nx, (d.nx & 3) == 0);
      }
    }
    // P(j - 3)'s operands (psi_q, K) into the slots P(j - 4) just consumed
    if (j + 1 - AS_L >= 0 && j + 1 - AS_L < nz) {
      psi_issue(psp, psq_p, j + 1 - AS_L);
      if (own) cp_async16(ksl, a.kk + (long long)(j + 1 - AS_L + GZ) * PS + oc);
    }
    cp_async_commit();
#pragma unroll
    for (int t = 0; t < 7; ++t) {
      r[t] = r[t + 1];
      zq[t] = zq[t + 1];
    }
    if (j < nz) {
      // ================================ V at plane j (kernels_acoustic.cuh ac_v, same arithmetic)
      const int s = j % AS_NSV;
      const int k = j;
      const long long o = (long long)(k + GZ) * PS + oc;
      const int gz = k + d.z0;
      const bool lz = Wl > 0 && CpmlIdx::in(gz, d.nz, Wl, a.zlo);
      if (lane == 0) AS_TRACE(k, 32 + (tid >> 5));  // every warp's V start (before the stage wait)
      mbar_wait(&fullv[s], (j / AS_NSV) & 1);
      if (tid == 0) AS_TRACE(k, 4);
      const float* st = smv + s * L::VSIZE;
      r[7] = lds4(st + L::PQ + pt);
      const F4 rz1 = lds4(st + L::RZ + pt);
      const float* c = st + L::PT + (ty + 4) * PW + 4 * tx + 4;  // p(x0, jy, k)
      float xv[12];
      {
        const F4 a0 = lds4(c - 4), a1 = lds4(c), a2 = lds4(c + 4);
#pragma unroll
        for (int e = 0; e < 4; ++e) {
          xv[e] = a0.v[e];
          xv[4 + e] = a1.v[e];
          xv[8 + e] = a2.v[e];
        }
      }
      F4 yr[8];  // p rows jy-3 .. jy+4
#pragma unroll
      for (int m = 0; m < 8; ++m) yr[m] = (m == 3) ? F4{{xv[4], xv[5], xv[6], xv[7]}} : lds4(c + (m - 3) * PW);
      float dx[4], dy[4], dz[4];
#pragma unroll
      for (int e = 0; e < 4; ++e) {
        float t = SEIS_D1 * (xv[5 + e] - xv[4 + e]);
        t = fmaf(SEIS_D2, xv[6 + e] - xv[3 + e], t);
        t = fmaf(SEIS_D3, xv[7 + e] - xv[2 + e], t);
        dx[e] = fmaf(SEIS_D4, xv[8 + e] - xv[1 + e], t);
        t = SEIS_D1 * (yr[4].v[e] - yr[3].v[e]);
        t = fmaf(SEIS_D2, yr[5].v[e] - yr[2].v[e], t);
        t = fmaf(SEIS_D3, yr[6].v[e] - yr[1].v[e], t);
        dy[e] = fmaf(SEIS_D4, yr[7].v[e] - yr[0].v[e], t);
        t = SEIS_D1 * (r[4].v[e] - r[3].v[e]);
        t = fmaf(SEIS_D2, r[5].v[e] - r[2].v[e], t);
        t = fmaf(SEIS_D3, r[6].v[e] - r[1].v[e], t);
        dz[e] = fmaf(SEIS_D4, r[7].v[e] - r[0].v[e], t);
      }
      F4 oz4{{0.f, 0.f, 0.f, 0.f}};
      cp_async_wait<1>();  // this thread's psi_p slots (V's group; P's younger may be pending)
      float* const psq = psq_v;
      if (own) {
        if (lx) {
          int ix[4];
          float ca[4], cb[4];
          psi_idx_x<4>(ix, d, Wl, x0, jy, k);
          const F4 ov = lds4(psq);
#pragma unroll
          for (int e = 0; e < 4; ++e) {
            ca[e] = cpt.x[2][4 * tx + e];
            cb[e] = cpt.x[3][4 * tx + e];
          }
          psi_upd_s<4>(dx, a.psx, ix, ov.v, ca, cb);
        }
        if (ly) {
          int iy[4];
          psi_idx_row<4>(iy, (k * (2 * Wl) + CpmlIdx::slot(jy, d.ny, Wl)) * d.nx + x0, x0, d.nx);
          const F4 ov = lds4(psq + QS);
          const float ya = cpt.y[2][ty], yb = cpt.y[3][ty];
          const float ca[4] = {ya, ya, ya, ya}, cb[4] = {yb, yb, yb, yb};
          if (vec4) psi_upd_v4(dy, a.psy, iy[0], ov.v, ca, cb);
          else psi_upd_s<4>(dy, a.psy, iy, ov.v, ca, cb);
        }
        if (lz) {
          int iz[4];
          psi_idx_row<4>(iz, (CpmlIdx::slot(gz, d.nz, Wl) * d.ny + jy) * d.nx + x0, x0, d.nx);
          const F4 ov = lds4(psq + 2 * QS);
          const float za = __ldg(a.cz.ah + gz), zb = __ldg(a.cz.bh + gz);
          const float ca[4] = {za, za, za, za}, cb[4] = {zb, zb, zb, zb};
          if (vec4) psi_upd_v4(dz, a.psz, iz[0], ov.v, ca, cb);
          else psi_upd_s<4>(dz, a.psz, iz, ov.v, ca, cb);
        }
        if (SEIS_AS_PSIPF && Wl > 0) {  // L2 prefetch of the memory variables AS_PF planes ahead
          psi_prefetch(psv, j + AS_PF);
          psi_prefetch(psp, j + AS_PF);
        }
        const F4 qxo = lds4(st + L::QX + pt), qyo = lds4(st + L::QY + pt), qzo = lds4(st + L::QZ + pt);
        const float* rc = st + L::R + ty * RW + 4 * tx;
        const F4 r0 = lds4(rc), rxn = lds4(rc + 4), ryn = lds4(rc + RW);
        const float rx5 = rxn.v[0];
        const bool zlast = gz + 1 >= d.nz;
        F4 oxq, oyq;
#pragma unroll
        for (int e = 0; e < 4; ++e) {
          const float rxp = (x0 + e + 1 < d.nx) ? (e < 3 ? r0.v[e + 1] : rx5) : r0.v[e];
          const float ryp = (jy + 1 < d.ny) ? ryn.v[e] : r0.v[e];
          const float rzp = zlast ? r0.v[e] : rz1.v[e];
          const float bx = dth * (2.0f * rcp_fast(r0.v[e] + rxp));
          const float by = dth * (2.0f * rcp_fast(r0.v[e] + ryp));
          const float bz = dth * (2.0f * rcp_fast(r0.v[e] + rzp));
          oxq.v[e] = fmaf(bx, dx[e], qxo.v[e]);
          oyq.v[e] = fmaf(by, dy[e], qyo.v[e]);
          oz4.v[e] = fmaf(bz, dz[e], qzo.v[e]);
        }
        st4_masked(a.qx + o, oxq, x0, d.nx, true);
        st4_masked(a.qy + o, oyq, x0, d.nx, true);
        st4_masked(a.qz + o, oz4, x0, d.nx, true);
        if (IMG) {
          const long long cix = ((long long)k * d.ny + jy) * d.nx + x0;
          F4 im;
#pragma unroll
          for (int e = 0; e < 4; ++e)
            im.v[e] = (x0 + e < d.nx) ? fmaf(a.imgR.at(cix + e), r[3].v[e], a.img[cix + e]) : 0.f;
          st4_masked(a.img + cix, im, x0, d.nx, false);
        }
#pragma unroll
        for (int e = 0; e < 4; ++e)
          if (x0 + e >= d.nx) oz4.v[e] = 0.f;  // (outside the grid q_z is a ghost zero, O1)
      }
      zq[7] = oz4;
      // release the stage -- after this warp's q stores: the producer publishes V(k) of the
      // tile once all warps arrived
      __syncwarp();
      if (lane == 0) mbar_arrive(&emptyv[s]);
      if (tid == 0) AS_TRACE(k, 5);
      if (tid == AS_CONS - 32) AS_TRACE(k, 7);
      if (lane == 0) AS_TRACE(k, 16 + (tid >> 5));  // every warp's V done
    } else {
      r[7] = F4{{0.f, 0.f, 0.f, 0.f}};
      zq[7] = F4{{0.f, 0.f, 0.f, 0.f}};
    }
  }
}

}  // namespace seis
