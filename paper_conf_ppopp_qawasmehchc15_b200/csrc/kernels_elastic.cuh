// kernels_elastic.cuh — Eq 3: isotropic elastic velocity-stress
// system on the staggered (Virieux) grid (O9), leapfrog (O2), C-PML (O7),
// stress-imaging free surface (O16).
//
// Grid (array index (i,j,k) of each field holds the position):
//   vx (i+1/2,j,k)  vy (i,j+1/2,k)  vz (i,j,k+1/2)   sxx syy szz (i,j,k)
//   sxy (i+1/2,j+1/2,k)  sxz (i+1/2,j,k+1/2)  syz (i,j+1/2,k+1/2)
// V:  vx += (dt b_x/h)(Dx+ sxx + Dy- sxy + Dz- sxz)   (+ psi 0,1,2)
//     vy += (dt b_y/h)(Dx- sxy + Dy+ syy + Dz- syz)   (+ psi 3,4,5)
//     vz += (dt b_z/h)(Dx- sxz + Dy- syz + Dz+ szz)   (+ psi 6,7,8)
// S:  exx = Dx- vx, eyy = Dy- vy, ezz = Dz- vz        (+ psi 9,10,11)
//     s_ii += (dt/h)[(lam + 2mu) e_ii + lam (sum of the other two)]
//     sxy += (dt mu_xy/h)(Dy+ vx + Dx+ vy)             (+ psi 12,13)
//     sxz += (dt mu_xz/h)(Dz+ vx + Dx+ vz)             (+ psi 14,15)
//     syz += (dt mu_yz/h)(Dz+ vy + Dy+ vz)             (+ psi 16,17)
// psi stored times h (unscaled differences).  Free surface (O16): the planes above
// k = 0 are the mirror images of the planes below (formed in the z-queue warm-up,
// ldg2_fs), the surface row uses ezz = -lam/(lam+2mu)(exx+eyy), and szz = 0 on
// k = 0 after the source.
//
// Both kernels are 2.5D z-marches over 64 x BY tiles with 2 x-points per thread
// (float2; each thread keeps three 8-deep z-queues in registers).  Every operand
// of plane k -- the halo tiles of the fields differentiated in x/y, the
// pointwise fields and coefficients, and the plane-(k+3|k+4) feeds of the
// z-queues -- arrives by TMA in one stage of an mbarrier ring.
#pragma once
#include "common.cuh"
#include "kernels_acoustic.cuh"  // CpmlAxis

namespace seis {

enum { EVX, EVY, EVZ, ESXX, ESYY, ESZZ, ESXY, ESXZ, ESYZ };

// staggered differences, times h, along a line of values v (index c = the point)
__device__ __forceinline__ float dp(const float* v, int c) {  // D+ at c+1/2 from integer field
  float r = SEIS_D1 * (v[c + 1] - v[c]);
  r = fmaf(SEIS_D2, v[c + 2] - v[c - 1], r);
  r = fmaf(SEIS_D3, v[c + 3] - v[c - 2], r);
  return fmaf(SEIS_D4, v[c + 4] - v[c - 3], r);
}
__device__ __forceinline__ float dm(const float* v, int c) {  // D- at c from half field
  float r = SEIS_D1 * (v[c] - v[c - 1]);
  r = fmaf(SEIS_D2, v[c + 1] - v[c - 2], r);
  r = fmaf(SEIS_D3, v[c + 2] - v[c - 3], r);
  return fmaf(SEIS_D4, v[c + 3] - v[c - 4], r);
}
// x-row of 10 values x0-4 .. x0+5 from a shared tile row (pointer at x0)
__device__ __forceinline__ void xrow(float* xv, const float* c) {
#pragma unroll
  for (int t = 0; t < 5; ++t) {
    const F2 a = lds2(c - 4 + 2 * t);
    xv[2 * t] = a.v[0];
    xv[2 * t + 1] = a.v[1];
  }
}
// y-column values rows j-4 .. j+4 (9) for the 2 components, from a tile (row stride S)
template <int S>
__device__ __forceinline__ void ycol(float (*yv)[9], const float* c) {
#pragma unroll
  for (int m = 0; m < 9; ++m) {
    const F2 a = lds2(c + (m - 4) * S);
    yv[0][m] = a.v[0];
    yv[1][m] = a.v[1];
  }
}

// z-queue warm-up load of plane p of field f at column offset oc.  With the free surface
// (O16), the planes above k = 0 of the top slab are the mirror images of the planes below
// it -- integer-z fields: plane -m = sgn f(m); half-z fields: plane -1-m = sgn f(m)
// (sgn = -1 for szz, sxz, syz) -- and they are only ever read here (every other operand of
// the z-march is at planes >= 0), so they are formed on the fly instead of being stored by
// a mirror kernel after every half step.
__device__ __forceinline__ F2 ldg2_fs(const float* __restrict__ f, int p, long long PS, long long oc, bool mirror,
                                      bool half, float sgn) {
  if (mirror && p < 0) {
    const F2 v = ldg2(f + (long long)((half ? -1 - p : -p) + GZ) * PS + oc);
    return F2{{sgn * v.v[0], sgn * v.v[1]}};
  }
  return ldg2(f + (long long)(p + GZ) * PS + oc);
}

// Warp specialization (default): one extra warp per block issues the TMA ring loads; consumer
// warps release a stage by arriving on its "empty" mbarrier, so no block-wide barrier remains
// in the z-march (ncu r01: 17 % of el_v's stalls were on the per-plane __syncthreads).  The
// block is then 32 x BY consumer threads + the producer warp, one block per SM (BY = 15:
// 16 warps, 128 registers per thread).  SEIS_EL_WS=0 restores the barrier-released ring.
#ifndef SEIS_EL_WS
#define SEIS_EL_WS 1
#endif
constexpr int EL_WS = SEIS_EL_WS;
// C-PML memory variables by cp.async (measured and rejected, off): the old values of plane
// k + 1 travel into per-thread shared slots (9 arrays x 2 points) while plane k computes,
// instead of being loaded into registers before the stage wait.  Correct (parity green) but
// el_v 0.734 vs 0.680 ms at C3 (the 4-byte cp.async issue + wait costs more than the register
// preload hides), and el_s needs a 2-stage ring to fit the slots (0.987 vs 0.886 ms);
// profiles/r02_el_psa_variants.log
#ifndef SEIS_EL_PSA
#define SEIS_EL_PSA 0
#endif
#ifndef SEIS_EL_VPSA
#define SEIS_EL_VPSA SEIS_EL_PSA
#endif
#ifndef SEIS_EL_SPSA
#define SEIS_EL_SPSA SEIS_EL_PSA
#endif
// (warp specialization) L2 prefetch distance of the producer, planes ahead of the ring loads
#ifndef SEIS_EL_PF
#define SEIS_EL_PF 0
#endif
constexpr int EL_PF = SEIS_EL_PF;
#ifndef SEIS_EL_PWAIT
#define SEIS_EL_PWAIT 1  // producer wait: 0 = test_wait + nanosleep, 1 = try_wait spin
#endif
#ifndef SEIS_EL_VNS
#define SEIS_EL_VNS 3
#endif
#ifndef SEIS_EL_SNS
#define SEIS_EL_SNS (SEIS_EL_WS ? 3 : 2)
#endif
#ifndef SEIS_EL_MINB
#define SEIS_EL_MINB 0  // launch-bounds minimum blocks per SM (0: 2 for BY <= 8, else 1)
#endif
constexpr int EL_VNS = SEIS_EL_VNS;
constexpr int EL_SNS = SEIS_EL_SNS;
// (C-PML body) L2 prefetch of the memory variables SEIS_EL_{V,S}PSIPF planes ahead, one lane
// per 128-byte slab line (0 = off).  Measured at C3 (profiles/r02_el_psipf.log): el_s 0.824 ->
// 0.812 ms at distance 2 (1: 0.814, 4: 0.934); el_v 0.650 -> 0.652 (no gain): S only.
#ifndef SEIS_EL_VPSIPF
#define SEIS_EL_VPSIPF 0
#endif
#ifndef SEIS_EL_SPSIPF
#define SEIS_EL_SPSIPF 2
#endif

// the L2 prefetch above: arrays X of the x slab [nzl][ny][2W], Y of the y slab [nzl][2W][nx],
// Z of the z slab [2W][ny][nx] at plane kk of this thread's row (lanes 0 / 16 of a warp row
// cover its 64 floats; the x-slab row is 2W contiguous floats)
template <int X0, int X1, int X2, int Y0, int Y1, int Y2, int Z0, int Z1, int Z2>
__device__ __forceinline__ void el_psi_prefetch(float* const* psi, const Dims& d, int W, int zlo, int tx, int x0,
                                                int j, bool lx, bool ly, int kk) {
  if (kk >= d.nzl) return;
  if (lx && (tx & 7) == 0) {
    const int b = (kk * d.ny + j) * (2 * W) + (x0 < W ? 0 : W);
    prefetch_l2(psi[X0] + b);
    prefetch_l2(psi[X1] + b);
    prefetch_l2(psi[X2] + b);
  }
  if ((tx & 15) != 0) return;
  if (ly) {
    const int b = (kk * (2 * W) + CpmlIdx::slot(j, d.ny, W)) * d.nx + x0;
    prefetch_l2(psi[Y0] + b);
    prefetch_l2(psi[Y1] + b);
    prefetch_l2(psi[Y2] + b);
  }
  const int gz = kk + d.z0;
  if (CpmlIdx::in(gz, d.nz, W, zlo)) {
    const int b = (CpmlIdx::slot(gz, d.nz, W) * d.ny + j) * d.nx + x0;
    prefetch_l2(psi[Z0] + b);
    prefetch_l2(psi[Z1] + b);
    prefetch_l2(psi[Z2] + b);
  }
}

struct ElVArgs {
  CUtensorMap msxx;   // box 72 x BY      (x halo)
  CUtensorMap msxy;   // box 72 x (BY+8)  (x and y halos)
  CUtensorMap msxz;   // box 72 x BY
  CUtensorMap msyy;   // box 64 x (BY+8)  (y halo)
  CUtensorMap msyz;   // box 64 x (BY+8)
  CUtensorMap mv[3];  // vx, vy, vz, box 64 x BY
  CUtensorMap mr;     // rho tile, box (64+4) x (BY+1) (x+1, y+1 neighbours)
  CUtensorMap mrz;    // rho interior at plane k+1, box 64 x BY
  CUtensorMap mq[3];  // z-queue feeds: sxz (k+3), syz (k+3), szz (k+4), box 64 x BY
  float* f[9];
  int W, zlo, fs;
  int region;  // 0: every block; 1: only blocks free of C-PML points; 2: only the others;
               // 3: every block, the lean body where no C-PML point is (one launch)
  float dth;       // dt / h (face buoyancy dt b/h = dth * 2/(rho_i + rho_{i+1}), O8/O9)
  CpmlAxis cx, cy, cz;
  float* psi[9];   // psi 0..8
  Dims d;
  int zc;
  int ch0, chs;                  // z-chunk of blockIdx.z = ch0 + blockIdx.z * chs (boundary / interior split)
  const float* __restrict__ imgS;  // elastic RTM (f3): img += S * P on the input level, P = -(sxx+syy+szz)/3
  SnapRef imgR;                    // the same (fp32 or 24-bit), what the IMG kernel reads
  float* __restrict__ img;
  Ghost gh[3];                     // direct ghost stores of vx, vy, vz (f4)
};

// (region split) may this block's tile (TXE x BY) and z-chunk hold a C-PML point
__device__ __forceinline__ bool el_block_in_layers(const Dims& d, int W, int zlo, int i0, int j0, int by, int k0,
                                                   int k1) {
  return block_in_layers(d, W, zlo, i0, TXE, j0, by, k0, k1);
}

template <int BY>
struct ElVStage {
  static constexpr int WX = TXE + 8, T = TXE * BY, RW = TXE + 4;
  static constexpr int XX = 0, XY = XX + r32(BY * WX), XZ = XY + r32((BY + 8) * WX), YY = XZ + r32(BY * WX),
                       YZ = YY + r32((BY + 8) * TXE), V = YZ + r32((BY + 8) * TXE), RZ = V + 3 * r32(T),
                       Q = RZ + r32(T), R = Q + 3 * r32(T), SIZE = R + r32(RW * (BY + 1));
  static constexpr int TS = r32(T);  // stride of the 3 v / 3 q tiles
  static constexpr uint32_t BYTES = (2 * BY * WX + (BY + 8) * WX + 2 * (BY + 8) * TXE + 7 * T + RW * (BY + 1)) * 4;
  static constexpr int PSLOT = 9 * NTX2 * BY * 2;  // per-thread C-PML slots (floats)
  static constexpr size_t smem_bytes() { return ((size_t)EL_VNS * SIZE + (SEIS_EL_VPSA ? PSLOT : 0)) * 4 + 128; }
};

template <int BY, bool IMG, bool CP>
__device__ __forceinline__ void el_v_body(const ElVArgs& a) {
  using L = ElVStage<BY>;
  constexpr int WX = L::WX;
  constexpr uint32_t TX_BYTES = L::BYTES;
  constexpr int RW = L::RW;
  static_assert((L::XY % 32) == 0 && (L::XZ % 32) == 0 && (L::YY % 32) == 0 && (L::V % 32) == 0 &&
                    (L::R % 32) == 0,
                "128-byte tiles");
  extern __shared__ __align__(128) float sm_raw[];
  float* sm = align128(sm_raw);
  __shared__ __align__(8) uint64_t bar[EL_VNS];
  __shared__ __align__(8) uint64_t ebar[EL_VNS];  // (warp specialization) stage consumed by all warps
  __shared__ uint32_t cnt[EL_VNS];
  __shared__ CpmlTile<TXE, BY> ctile;  // x / y C-PML coefficients of this tile
  const Dims& d = a.d;
  const int tx = threadIdx.x, ty = threadIdx.y, tid = ty * NTX2 + tx;
  const int i0 = blockIdx.x * TXE, j0 = blockIdx.y * BY;
  const int x0 = i0 + 2 * tx, j = j0 + ty;
  const int k0 = (a.ch0 + (int)blockIdx.z * a.chs) * a.zc;
  const int k1 = min(k0 + a.zc, d.nzl);
  const int np = k1 - k0;
  const bool own = (x0 < d.nx) && (j < d.ny);
  const long long PS = d.PS;
  const long long oc = (long long)(j + G) * d.PX + (x0 + G);
  // (region split) CP = false: the instantiation without the C-PML code, for blocks whose
  // tile and z-chunk hold no layer point (fewer instructions, no spills)
  if ((a.region == 1 || a.region == 2) && el_block_in_layers(d, a.W, a.zlo, i0, j0, BY, k0, k1) != (a.region == 2))
    return;
  const int W = CP ? a.W : 0;
  const bool lx = W > 0 && (x0 < W || x0 + 1 >= d.nx - W);
  const bool ly = W > 0 && CpmlIdx::in(j, d.ny, W, true);
  auto issue = [&](int s, int k, bool pf = false) {
    float* st = sm + s * L::SIZE;
    const int z = k + GZ, x = i0 + G, y = j0 + G;
    if (!pf) mbar_expect_tx(&bar[s], TX_BYTES);
    tma_ld(pf, st + L::XX, &a.msxx, &bar[s], i0, y, z);
    tma_ld(pf, st + L::XY, &a.msxy, &bar[s], i0, j0, z);
    tma_ld(pf, st + L::XZ, &a.msxz, &bar[s], i0, y, z);
    tma_ld(pf, st + L::YY, &a.msyy, &bar[s], x, j0, z);
    tma_ld(pf, st + L::YZ, &a.msyz, &bar[s], x, j0, z);
#pragma unroll
    for (int c = 0; c < 3; ++c) tma_ld(pf, st + L::V + c * L::TS, &a.mv[c], &bar[s], x, y, z);
    tma_ld(pf, st + L::R, &a.mr, &bar[s], x, y, z);
    tma_ld(pf, st + L::RZ, &a.mrz, &bar[s], x, y, z + 1);
    tma_ld(pf, st + L::Q, &a.mq[0], &bar[s], x, y, z + 3);
    tma_ld(pf, st + L::Q + L::TS, &a.mq[1], &bar[s], x, y, z + 3);
    tma_ld(pf, st + L::Q + 2 * L::TS, &a.mq[2], &bar[s], x, y, z + 4);
  };
  if (tid == 0) {
    for (int s = 0; s < EL_VNS; ++s) {
      mbar_init(&bar[s], 1);
      mbar_init(&ebar[s], BY);
      cnt[s] = 0u;
    }
    mbar_fence_init();
  }
  cpml_tile_fill(ctile, a.cx, a.cy, blockIdx.x * TXE, blockIdx.y * BY, a.d.nx, a.d.ny, W > 0, tid,
                 NTX2 * (BY + EL_WS));
  __syncthreads();
  if (EL_WS && ty == BY) {  // producer warp: lane 0 refills each stage once all warps released it
    if (tx == 0)
      for (int it = 0; it < np; ++it) {
        const int s = it % EL_VNS;
        if (it >= EL_VNS) {
          if (SEIS_EL_PWAIT) mbar_wait(&ebar[s], ((it / EL_VNS) - 1) & 1);
          else mbar_wait_nap(&ebar[s], ((it / EL_VNS) - 1) & 1);
        }
        issue(s, k0 + it);
        if (EL_PF > 0 && it + EL_PF < np) issue(s, k0 + it + EL_PF, true);  // L2 prefetch
      }
    return;
  }
  if (!EL_WS && tid == 0)
    for (int s = 0; s < EL_VNS && s < np; ++s) issue(s, k0 + s);
  if (!EL_WS && tid == 0)
    for (int t = 0; t < L2PF && EL_VNS + t < np; ++t) issue(0, k0 + EL_VNS + t, true);
  // (C-PML by cp.async) per-thread slots of the 9 memory variables of plane kk (2 points each)
  float* const psl = sm + EL_VNS * L::SIZE + 2 * tid;
  constexpr int PST = NTX2 * BY * 2;  // slot stride of one array
  auto psi_issue = [&](int kk) {
    const int gzk = kk + d.z0;
    int ix[2];
    if (own && lx) {
      psi_idx_x<2>(ix, d, W, x0, j, kk);
#pragma unroll
      for (int e = 0; e < 2; ++e)
        if (ix[e] >= 0)
          for (int t : {0, 3, 6}) cp_async4(psl + t * PST + e, a.psi[t] + ix[e], true);
    }
    if (own && ly) {
      psi_idx_row<2>(ix, (kk * (2 * W) + CpmlIdx::slot(j, d.ny, W)) * d.nx + x0, x0, d.nx);
#pragma unroll
      for (int e = 0; e < 2; ++e)
        if (ix[e] >= 0)
          for (int t : {1, 4, 7}) cp_async4(psl + t * PST + e, a.psi[t] + ix[e], true);
    }
    if (own && W > 0 && CpmlIdx::in(gzk, d.nz, W, a.zlo)) {
      psi_idx_row<2>(ix, (CpmlIdx::slot(gzk, d.nz, W) * d.ny + j) * d.nx + x0, x0, d.nx);
#pragma unroll
      for (int e = 0; e < 2; ++e)
        if (ix[e] >= 0)
          for (int t : {2, 5, 8}) cp_async4(psl + t * PST + e, a.psi[t] + ix[e], true);
    }
    cp_async_commit();
  };
  if (SEIS_EL_VPSA && W > 0 && np > 0) psi_issue(k0);
  const float* __restrict__ sxz = a.f[ESXZ];
  const float* __restrict__ syz = a.f[ESYZ];
  const float* __restrict__ szz = a.f[ESZZ];
  F2 qxz[8], qyz[8], qzz[8];  // sxz, syz at k-4..k+3 (D-); szz at k-3..k+4 (D+)
  if (a.fs && d.z0 == 0 && k0 < 4) {  // free-surface images above the top slab (O16)
#pragma unroll
    for (int t = 0; t < 7; ++t) {
      qxz[t] = ldg2_fs(sxz, k0 - 4 + t, PS, oc, true, true, -1.0f);
      qyz[t] = ldg2_fs(syz, k0 - 4 + t, PS, oc, true, true, -1.0f);
      qzz[t] = ldg2_fs(szz, k0 - 3 + t, PS, oc, true, false, -1.0f);
    }
  } else {
#pragma unroll
    for (int t = 0; t < 7; ++t) {
      qxz[t] = ldg2(sxz + (long long)(k0 - 4 + t + GZ) * PS + oc);
      qyz[t] = ldg2(syz + (long long)(k0 - 4 + t + GZ) * PS + oc);
      qzz[t] = ldg2(szz + (long long)(k0 - 3 + t + GZ) * PS + oc);
    }
  }
  // does this slab store ghost planes of a neighbour (f4)?
  const bool ghk = a.gh[0].lo || a.gh[0].hi || a.gh[1].lo || a.gh[1].hi || a.gh[2].lo || a.gh[2].hi;
  SEIS_UNROLL(SEIS_ZU_EL)
  for (int it = 0; it < np; ++it) {
    const int k = k0 + it;
    const int s = it % EL_VNS;
    const long long o = (long long)(k + GZ) * PS + oc;
    // C-PML: old psi values are loaded before the wait (latency overlap)
    const int gz = k + d.z0;
    const bool lz = W > 0 && CpmlIdx::in(gz, d.nz, W, a.zlo);
    int ixx[2], iyy[2], izz[2];  // 32-bit compact-slab indices (fewer live registers)
    float ox0[2], ox3[2], ox6[2], oy1[2], oy4[2], oy7[2], oz2[2], oz5[2], oz8[2];
    if (!SEIS_EL_VPSA && own && lx) {
      psi_idx_x<2>(ixx, d, W, x0, j, k);
      psi_ld<2>(ox0, a.psi[0], ixx);
      psi_ld<2>(ox3, a.psi[3], ixx);
      psi_ld<2>(ox6, a.psi[6], ixx);
    }
    if (!SEIS_EL_VPSA && own && ly) {
      psi_idx_row<2>(iyy, (k * (2 * W) + CpmlIdx::slot(j, d.ny, W)) * d.nx + x0, x0, d.nx);
      psi_ld<2>(oy1, a.psi[1], iyy);
      psi_ld<2>(oy4, a.psi[4], iyy);
      psi_ld<2>(oy7, a.psi[7], iyy);
    }
    if (!SEIS_EL_VPSA && own && lz) {
      psi_idx_row<2>(izz, (CpmlIdx::slot(gz, d.nz, W) * d.ny + j) * d.nx + x0, x0, d.nx);
      psi_ld<2>(oz2, a.psi[2], izz);
      psi_ld<2>(oz5, a.psi[5], izz);
      psi_ld<2>(oz8, a.psi[8], izz);
    }
    if (SEIS_EL_VPSIPF > 0 && W > 0 && own)
      el_psi_prefetch<0, 3, 6, 1, 4, 7, 2, 5, 8>(a.psi, d, W, a.zlo, tx, x0, j, lx, ly, k + SEIS_EL_VPSIPF);
    mbar_wait(&bar[s], (it / EL_VNS) & 1);
    const float* st = sm + s * L::SIZE;
    const int pt = ty * TXE + 2 * tx;
    qxz[7] = lds2(st + L::Q + pt);
    qyz[7] = lds2(st + L::Q + L::TS + pt);
    qzz[7] = lds2(st + L::Q + 2 * L::TS + pt);
    if (own) {
      float xs[10], xy[10], xz[10], yxy[2][9], yyy[2][9], yyz[2][9];
      xrow(xs, st + L::XX + ty * WX + 2 * tx + 4);
      xrow(xy, st + L::XY + (ty + 4) * WX + 2 * tx + 4);
      xrow(xz, st + L::XZ + ty * WX + 2 * tx + 4);
      ycol<WX>(yxy, st + L::XY + (ty + 4) * WX + 2 * tx + 4);
      ycol<TXE>(yyy, st + L::YY + (ty + 4) * TXE + 2 * tx);
      ycol<TXE>(yyz, st + L::YZ + (ty + 4) * TXE + 2 * tx);
      float d0[2], d1[2], d2[2], d3[2], d4[2], d5[2], d6[2], d7[2], d8[2];
#pragma unroll
      for (int e = 0; e < 2; ++e) {
        float zxz[8], zyz[8], zzz[8];
#pragma unroll
        for (int t = 0; t < 8; ++t) {
          zxz[t] = qxz[t].v[e];
          zyz[t] = qyz[t].v[e];
          zzz[t] = qzz[t].v[e];
        }
        d0[e] = dp(xs, 4 + e);   // Dx+ sxx
        d1[e] = dm(yxy[e], 4);   // Dy- sxy
        d2[e] = dm(zxz, 4);      // Dz- sxz  (zxz[0..7] = k-4..k+3)
        d3[e] = dm(xy, 4 + e);   // Dx- sxy
        d4[e] = dp(yyy[e], 4);   // Dy+ syy
        d5[e] = dm(zyz, 4);      // Dz- syz
        d6[e] = dm(xz, 4 + e);   // Dx- sxz
        d7[e] = dm(yyz[e], 4);   // Dy- syz
        d8[e] = dp(zzz, 3);      // Dz+ szz  (zzz[0..7] = k-3..k+4)
      }
      if (SEIS_EL_VPSA && W > 0) {  // the slots of this plane (issued one plane ahead)
        cp_async_wait<0>();
        if (lx) {
          psi_idx_x<2>(ixx, d, W, x0, j, k);
          { const F2 v = lds2(psl + 0 * PST); ox0[0] = v.v[0]; ox0[1] = v.v[1]; }
          { const F2 v = lds2(psl + 3 * PST); ox3[0] = v.v[0]; ox3[1] = v.v[1]; }
          { const F2 v = lds2(psl + 6 * PST); ox6[0] = v.v[0]; ox6[1] = v.v[1]; }
        }
        if (ly) {
          psi_idx_row<2>(iyy, (k * (2 * W) + CpmlIdx::slot(j, d.ny, W)) * d.nx + x0, x0, d.nx);
          { const F2 v = lds2(psl + 1 * PST); oy1[0] = v.v[0]; oy1[1] = v.v[1]; }
          { const F2 v = lds2(psl + 4 * PST); oy4[0] = v.v[0]; oy4[1] = v.v[1]; }
          { const F2 v = lds2(psl + 7 * PST); oy7[0] = v.v[0]; oy7[1] = v.v[1]; }
        }
        if (lz) {
          psi_idx_row<2>(izz, (CpmlIdx::slot(gz, d.nz, W) * d.ny + j) * d.nx + x0, x0, d.nx);
          { const F2 v = lds2(psl + 2 * PST); oz2[0] = v.v[0]; oz2[1] = v.v[1]; }
          { const F2 v = lds2(psl + 5 * PST); oz5[0] = v.v[0]; oz5[1] = v.v[1]; }
          { const F2 v = lds2(psl + 8 * PST); oz8[0] = v.v[0]; oz8[1] = v.v[1]; }
        }
      }
      if (lx) {
        float ca[2], cb[2], cah[2], cbh[2];
#pragma unroll
        for (int e = 0; e < 2; ++e) {
          const int c = min(x0 + e, d.nx - 1) - i0;
          ca[e] = ctile.x[0][c]; cb[e] = ctile.x[1][c];
          cah[e] = ctile.x[2][c]; cbh[e] = ctile.x[3][c];
        }
        psi_upd<2>(d0, a.psi[0], ixx, ox0, cah, cbh);
        psi_upd<2>(d3, a.psi[3], ixx, ox3, ca, cb);
        psi_upd<2>(d6, a.psi[6], ixx, ox6, ca, cb);
      }
      if (ly) {
        const float ya = ctile.y[0][ty], yb = ctile.y[1][ty];
        const float yah = ctile.y[2][ty], ybh = ctile.y[3][ty];
        const float ca[2] = {ya, ya}, cb[2] = {yb, yb}, cah[2] = {yah, yah}, cbh[2] = {ybh, ybh};
        psi_upd<2>(d1, a.psi[1], iyy, oy1, ca, cb);
        psi_upd<2>(d4, a.psi[4], iyy, oy4, cah, cbh);
        psi_upd<2>(d7, a.psi[7], iyy, oy7, ca, cb);
      }
      if (lz) {
        const float za = __ldg(a.cz.a + gz), zb = __ldg(a.cz.b + gz);
        const float zah = __ldg(a.cz.ah + gz), zbh = __ldg(a.cz.bh + gz);
        const float ca[2] = {za, za}, cb[2] = {zb, zb}, cah[2] = {zah, zah}, cbh[2] = {zbh, zbh};
        psi_upd<2>(d2, a.psi[2], izz, oz2, ca, cb);
        psi_upd<2>(d5, a.psi[5], izz, oz5, ca, cb);
        psi_upd<2>(d8, a.psi[8], izz, oz8, cah, cbh);
      }
      const F2 v0 = lds2(st + L::V + pt), v1 = lds2(st + L::V + L::TS + pt), v2 = lds2(st + L::V + 2 * L::TS + pt);
      // face buoyancy dt b/h = (dt/h) 2/(rho_i + rho_{i+1}), the last face clamps (O8, O9)
      const float* rc = st + L::R + ty * RW + 2 * tx;
      const F2 r0 = lds2(rc), ryn = lds2(rc + RW), rzn = lds2(st + L::RZ + pt);
      const float rx2 = lds2(rc + 2).v[0];  // (8-byte load: no 2-way bank conflict)
      const bool zlast = k + d.z0 + 1 >= d.nz;
      F2 ov[3];
#pragma unroll
      for (int e = 0; e < 2; ++e) {
        const float rxp = (x0 + e + 1 < d.nx) ? (e == 0 ? r0.v[1] : rx2) : r0.v[e];
        const float ryp = (j + 1 < d.ny) ? ryn.v[e] : r0.v[e];
        const float rzp = zlast ? r0.v[e] : rzn.v[e];
        const float bx = a.dth * (2.0f * rcp_fast(r0.v[e] + rxp));
        const float by = a.dth * (2.0f * rcp_fast(r0.v[e] + ryp));
        const float bz = a.dth * (2.0f * rcp_fast(r0.v[e] + rzp));
        ov[0].v[e] = fmaf(bx, (d0[e] + d1[e]) + d2[e], v0.v[e]);
        ov[1].v[e] = fmaf(by, (d3[e] + d4[e]) + d5[e], v1.v[e]);
        ov[2].v[e] = fmaf(bz, (d6[e] + d7[e]) + d8[e], v2.v[e]);
      }
      // one x-bound branch for the 3 stores (a branch per store cost a reconvergence pair each);
      // the ghost-store tests only on the 4 boundary planes of a slab that has a neighbour
      if (x0 + 1 < d.nx) {
#pragma unroll
        for (int c = 0; c < 3; ++c) *reinterpret_cast<float2*>(a.f[EVX + c] + o) = make_float2(ov[c].v[0], ov[c].v[1]);
      } else {
#pragma unroll
        for (int c = 0; c < 3; ++c) a.f[EVX + c][o] = ov[c].v[0];
      }
      if (ghk && (k < 4 || k >= d.nzl - 4)) {
#pragma unroll
        for (int c = 0; c < 3; ++c) ghost_st2(a.gh[c], o, k, d.nzl, ov[c], x0, d.nx);
      }
      if (IMG) {
        const long long cix = ((long long)k * d.ny + j) * d.nx + x0;
#pragma unroll
        for (int e = 0; e < 2; ++e)
          if (x0 + e < d.nx) {
            const float pr = -((xs[4 + e] + yyy[e][4]) + qzz[3].v[e]) / 3.0f;
            a.img[cix + e] = fmaf(a.imgR.at(cix + e), pr, a.img[cix + e]);
          }
      }
    }
    if (SEIS_EL_VPSA && W > 0 && it + 1 < np) psi_issue(k + 1);  // (own slots are consumed)
    if (EL_WS) {
      __syncwarp();
      if (tx == 0) mbar_arrive(&ebar[s]);
    } else {
      stage_release<(SEIS_WR_EL != 0)>(&cnt[s], tid, it + EL_VNS < np, [&] {
        issue(s, k + EL_VNS);
        if (L2PF && it + EL_VNS + L2PF < np) issue(s, k + EL_VNS + L2PF, true);
      });
    }
#pragma unroll
    for (int t = 0; t < 7; ++t) {
      qxz[t] = qxz[t + 1];
      qyz[t] = qyz[t + 1];
      qzz[t] = qzz[t + 1];
    }
  }
}

// (region = 3) one launch, the code path chosen per block: blocks whose tile and z-chunk hold
// no C-PML point run the body without the memory-variable code (as the lean instantiation)
template <int BY, bool IMG, bool CP>
__global__ void __launch_bounds__(NTX2 *(BY + EL_WS), SEIS_EL_MINB > 0 ? SEIS_EL_MINB : (BY <= 8 ? 2 : 1)) el_v_kernel(const __grid_constant__ ElVArgs a) {
  if (CP && a.region == 3) {
    const int k0 = (a.ch0 + (int)blockIdx.z * a.chs) * a.zc;
    const int k1 = min(k0 + a.zc, a.d.nzl);
    if (!el_block_in_layers(a.d, a.W, a.zlo, blockIdx.x * TXE, blockIdx.y * BY, BY, k0, k1)) {
      el_v_body<BY, IMG, false>(a);
      return;
    }
  }
  el_v_body<BY, IMG, CP>(a);
}

struct ElSArgs {
  CUtensorMap mvt[3];  // vx, vy, vz tiles, box 72 x (BY+8)
  CUtensorMap ms[6];   // sxx, syy, szz, sxy, sxz, syz, box 64 x BY
  CUtensorMap ml2m;    // dt (lam + 2 mu) / h, box 64 x BY
  CUtensorMap mw;      // w = h / (dt mu) (+inf where mu = 0), box (64+4) x (BY+1), planes k, k+1
  CUtensorMap mq[3];   // z-queue feeds: vx (k+4), vy (k+4), vz (k+3), box 64 x BY
  float* f[9];
  int W, zlo, fs;
  int region;  // 0: every block; 1: only blocks free of C-PML points; 2: only the others;
               // 3: every block, the lean body where no C-PML point is (one launch)
  CpmlAxis cx, cy, cz;
  float* psi[9];   // psi 9..17
  Dims d;
  int zc;
  int ch0, chs;                  // z-chunk of blockIdx.z = ch0 + blockIdx.z * chs (boundary / interior split)
  long long src_o;
  SrcAmp src;      // dt (lam + 2/3 mu)_s / h^3 * s[n]
  float* __restrict__ snap;  // elastic RTM (f3): snapshot of P = -(sxx+syy+szz)/3, or nullptr
  Ghost gh[3];               // direct ghost stores of szz, sxz, syz (f4)
};

template <int BY>
struct ElSStage {
  static constexpr int WX = TXE + 8, T = TXE * BY, TV = r32((BY + 8) * WX), RW = TXE + 4, TS = r32(TXE * BY);
  static constexpr int WT = ((RW * (BY + 1) + 31) / 32) * 32;
  static constexpr int VT = 0, S = 3 * TV, C = S + 6 * TS, Q = C + TS, WK = Q + 3 * TS, WK1 = WK + WT,
                       SIZE = WK1 + WT;
  static constexpr uint32_t BYTES = (3 * (BY + 8) * WX + 10 * T + 2 * RW * (BY + 1)) * 4;  // what the TMA boxes deliver
  static constexpr int PSLOT = 9 * NTX2 * BY * 2;  // per-thread C-PML slots (floats)
  static constexpr size_t smem_bytes() { return ((size_t)EL_SNS * SIZE + (SEIS_EL_SPSA ? PSLOT : 0)) * 4 + 128; }
};

template <int BY, bool SNAP, bool CP>
__device__ __forceinline__ void el_s_body(const ElSArgs& a) {
  using L = ElSStage<BY>;
  constexpr int WX = L::WX, TV = L::TV, RW = L::RW;
  constexpr uint32_t TX_BYTES = L::BYTES;
  static_assert((L::S % 32) == 0 && (L::C % 32) == 0 && (L::WK % 32) == 0 && (L::WK1 % 32) == 0,
                "128-byte tiles");
  extern __shared__ __align__(128) float sm_raw[];
  float* sm = align128(sm_raw);
  __shared__ __align__(8) uint64_t bar[EL_SNS];
  __shared__ __align__(8) uint64_t ebar[EL_SNS];  // (warp specialization) stage consumed by all warps
  __shared__ uint32_t cnt[EL_SNS];
  __shared__ CpmlTile<TXE, BY> ctile;  // x / y C-PML coefficients of this tile
  const Dims& d = a.d;
  const int tx = threadIdx.x, ty = threadIdx.y, tid = ty * NTX2 + tx;
  const int i0 = blockIdx.x * TXE, j0 = blockIdx.y * BY;
  const int x0 = i0 + 2 * tx, j = j0 + ty;
  const int k0 = (a.ch0 + (int)blockIdx.z * a.chs) * a.zc;
  const int k1 = min(k0 + a.zc, d.nzl);
  const int np = k1 - k0;
  const bool own = (x0 < d.nx) && (j < d.ny);
  const long long PS = d.PS;
  const long long oc = (long long)(j + G) * d.PX + (x0 + G);
  // (region split) CP = false: the instantiation without the C-PML code, for blocks whose
  // tile and z-chunk hold no layer point (fewer instructions, no spills)
  if ((a.region == 1 || a.region == 2) && el_block_in_layers(d, a.W, a.zlo, i0, j0, BY, k0, k1) != (a.region == 2))
    return;
  const int W = CP ? a.W : 0;
  const bool lx = W > 0 && (x0 < W || x0 + 1 >= d.nx - W);
  const bool ly = W > 0 && CpmlIdx::in(j, d.ny, W, true);
  auto issue = [&](int s, int k, bool pf = false) {
    float* st = sm + s * L::SIZE;
    const int z = k + GZ, x = i0 + G, y = j0 + G;
    if (!pf) mbar_expect_tx(&bar[s], TX_BYTES);
#pragma unroll
    for (int c = 0; c < 3; ++c) tma_ld(pf, st + L::VT + c * TV, &a.mvt[c], &bar[s], i0, j0, z);
#pragma unroll
    for (int c = 0; c < 6; ++c) tma_ld(pf, st + L::S + c * L::TS, &a.ms[c], &bar[s], x, y, z);
    tma_ld(pf, st + L::C, &a.ml2m, &bar[s], x, y, z);
    tma_ld(pf, st + L::WK, &a.mw, &bar[s], x, y, z);
    tma_ld(pf, st + L::WK1, &a.mw, &bar[s], x, y, z + 1);
    tma_ld(pf, st + L::Q, &a.mq[0], &bar[s], x, y, z + 4);
    tma_ld(pf, st + L::Q + L::TS, &a.mq[1], &bar[s], x, y, z + 4);
    tma_ld(pf, st + L::Q + 2 * L::TS, &a.mq[2], &bar[s], x, y, z + 3);
  };
  if (tid == 0) {
    for (int s = 0; s < EL_SNS; ++s) {
      mbar_init(&bar[s], 1);
      mbar_init(&ebar[s], BY);
      cnt[s] = 0u;
    }
    mbar_fence_init();
  }
  cpml_tile_fill(ctile, a.cx, a.cy, blockIdx.x * TXE, blockIdx.y * BY, a.d.nx, a.d.ny, W > 0, tid,
                 NTX2 * (BY + EL_WS));
  __syncthreads();
  if (EL_WS && ty == BY) {  // producer warp: lane 0 refills each stage once all warps released it
    if (tx == 0)
      for (int it = 0; it < np; ++it) {
        const int s = it % EL_SNS;
        if (it >= EL_SNS) {
          if (SEIS_EL_PWAIT) mbar_wait(&ebar[s], ((it / EL_SNS) - 1) & 1);
          else mbar_wait_nap(&ebar[s], ((it / EL_SNS) - 1) & 1);
        }
        issue(s, k0 + it);
        if (EL_PF > 0 && it + EL_PF < np) issue(s, k0 + it + EL_PF, true);  // L2 prefetch
      }
    return;
  }
  if (!EL_WS && tid == 0)
    for (int s = 0; s < EL_SNS && s < np; ++s) issue(s, k0 + s);
  if (!EL_WS && tid == 0)
    for (int t = 0; t < L2PF && EL_SNS + t < np; ++t) issue(0, k0 + EL_SNS + t, true);
  // (C-PML by cp.async) per-thread slots of the 9 memory variables of plane kk (2 points each)
  float* const psl = sm + EL_SNS * L::SIZE + 2 * tid;
  constexpr int PST = NTX2 * BY * 2;  // slot stride of one array
  auto psi_issue = [&](int kk) {
    const int gzk = kk + d.z0;
    int ix[2];
    if (own && lx) {
      psi_idx_x<2>(ix, d, W, x0, j, kk);
#pragma unroll
      for (int e = 0; e < 2; ++e)
        if (ix[e] >= 0)
          for (int t : {0, 4, 6}) cp_async4(psl + t * PST + e, a.psi[t] + ix[e], true);
    }
    if (own && ly) {
      psi_idx_row<2>(ix, (kk * (2 * W) + CpmlIdx::slot(j, d.ny, W)) * d.nx + x0, x0, d.nx);
#pragma unroll
      for (int e = 0; e < 2; ++e)
        if (ix[e] >= 0)
          for (int t : {1, 3, 8}) cp_async4(psl + t * PST + e, a.psi[t] + ix[e], true);
    }
    if (own && W > 0 && CpmlIdx::in(gzk, d.nz, W, a.zlo)) {
      psi_idx_row<2>(ix, (CpmlIdx::slot(gzk, d.nz, W) * d.ny + j) * d.nx + x0, x0, d.nx);
#pragma unroll
      for (int e = 0; e < 2; ++e)
        if (ix[e] >= 0)
          for (int t : {2, 5, 7}) cp_async4(psl + t * PST + e, a.psi[t] + ix[e], true);
    }
    cp_async_commit();
  };
  if (SEIS_EL_SPSA && W > 0 && np > 0) psi_issue(k0);
  const float* __restrict__ vx = a.f[EVX];
  const float* __restrict__ vy = a.f[EVY];
  const float* __restrict__ vz = a.f[EVZ];
  F2 qx[8], qy[8], qz[8];  // vx, vy at k-3..k+4 (D+); vz at k-4..k+3 (D-)
  if (a.fs && d.z0 == 0 && k0 < 4) {  // free-surface images above the top slab (O16)
#pragma unroll
    for (int t = 0; t < 7; ++t) {
      qx[t] = ldg2_fs(vx, k0 - 3 + t, PS, oc, true, false, 1.0f);
      qy[t] = ldg2_fs(vy, k0 - 3 + t, PS, oc, true, false, 1.0f);
      qz[t] = ldg2_fs(vz, k0 - 4 + t, PS, oc, true, true, 1.0f);
    }
  } else {
#pragma unroll
    for (int t = 0; t < 7; ++t) {
      qx[t] = ldg2(vx + (long long)(k0 - 3 + t + GZ) * PS + oc);
      qy[t] = ldg2(vy + (long long)(k0 - 3 + t + GZ) * PS + oc);
      qz[t] = ldg2(vz + (long long)(k0 - 4 + t + GZ) * PS + oc);
    }
  }
  // (the per-plane 64-bit source test stays here: src_hit measured slower in this kernel,
  // el_s 0.847 vs 0.821 ms, profiles/r02_src_store_ab.log)
  const long long srel0 = a.src_o - oc;
  // does this slab store ghost planes of a neighbour (f4)?
  const bool ghk = a.gh[0].lo || a.gh[0].hi || a.gh[1].lo || a.gh[1].hi || a.gh[2].lo || a.gh[2].hi;
  SEIS_UNROLL(SEIS_ZU_EL)
  for (int it = 0; it < np; ++it) {
    const int k = k0 + it;
    const int s = it % EL_SNS;
    const long long o = (long long)(k + GZ) * PS + oc;
    // C-PML: old psi values are loaded before the wait (latency overlap)
    const int gz = k + d.z0;
    const bool lz = W > 0 && CpmlIdx::in(gz, d.nz, W, a.zlo);
    int ixx[2], iyy[2], izz[2];  // 32-bit compact-slab indices (fewer live registers)
    float ox0[2], ox4[2], ox6[2], oy1[2], oy3[2], oy8[2], oz2[2], oz5[2], oz7[2];
    if (!SEIS_EL_SPSA && own && lx) {
      psi_idx_x<2>(ixx, d, W, x0, j, k);
      psi_ld<2>(ox0, a.psi[0], ixx);
      psi_ld<2>(ox4, a.psi[4], ixx);
      psi_ld<2>(ox6, a.psi[6], ixx);
    }
    if (!SEIS_EL_SPSA && own && ly) {
      psi_idx_row<2>(iyy, (k * (2 * W) + CpmlIdx::slot(j, d.ny, W)) * d.nx + x0, x0, d.nx);
      psi_ld<2>(oy1, a.psi[1], iyy);
      psi_ld<2>(oy3, a.psi[3], iyy);
      psi_ld<2>(oy8, a.psi[8], iyy);
    }
    if (!SEIS_EL_SPSA && own && lz) {
      psi_idx_row<2>(izz, (CpmlIdx::slot(gz, d.nz, W) * d.ny + j) * d.nx + x0, x0, d.nx);
      psi_ld<2>(oz2, a.psi[2], izz);
      psi_ld<2>(oz5, a.psi[5], izz);
      psi_ld<2>(oz7, a.psi[7], izz);
    }
    if (SEIS_EL_SPSIPF > 0 && W > 0 && own)
      el_psi_prefetch<0, 4, 6, 1, 3, 8, 2, 5, 7>(a.psi, d, W, a.zlo, tx, x0, j, lx, ly, k + SEIS_EL_SPSIPF);
    mbar_wait(&bar[s], (it / EL_SNS) & 1);
    const float* st = sm + s * L::SIZE;
    const int pt = ty * TXE + 2 * tx;
    qx[7] = lds2(st + L::Q + pt);
    qy[7] = lds2(st + L::Q + L::TS + pt);
    qz[7] = lds2(st + L::Q + 2 * L::TS + pt);
    if (own) {
      const float* cvx = st + L::VT + (ty + 4) * WX + 2 * tx + 4;
      const float* cvy = cvx + TV;
      const float* cvz = cvx + 2 * TV;
      float xvx[10], xvy[10], xvz[10], yvx[2][9], yvy[2][9], yvz[2][9];
      xrow(xvx, cvx);
      xrow(xvy, cvy);
      xrow(xvz, cvz);
      ycol<WX>(yvx, cvx);
      ycol<WX>(yvy, cvy);
      ycol<WX>(yvz, cvz);
      float exx[2], eyy[2], ezz[2], dyvx[2], dxvy[2], dzvx[2], dxvz[2], dzvy[2], dyvz[2];
#pragma unroll
      for (int e = 0; e < 2; ++e) {
        float zx[8], zy[8], zz[8];
#pragma unroll
        for (int t = 0; t < 8; ++t) {
          zx[t] = qx[t].v[e];
          zy[t] = qy[t].v[e];
          zz[t] = qz[t].v[e];
        }
        exx[e] = dm(xvx, 4 + e);   // Dx- vx
        eyy[e] = dm(yvy[e], 4);    // Dy- vy
        ezz[e] = dm(zz, 4);        // Dz- vz  (zz[0..7] = k-4..k+3)
        dyvx[e] = dp(yvx[e], 4);   // Dy+ vx
        dxvy[e] = dp(xvy, 4 + e);  // Dx+ vy
        dzvx[e] = dp(zx, 3);       // Dz+ vx  (zx[0..7] = k-3..k+4)
        dxvz[e] = dp(xvz, 4 + e);  // Dx+ vz
        dzvy[e] = dp(zy, 3);       // Dz+ vy
        dyvz[e] = dp(yvz[e], 4);   // Dy+ vz
      }
      if (SEIS_EL_SPSA && W > 0) {  // the slots of this plane (issued one plane ahead)
        cp_async_wait<0>();
        if (lx) {
          psi_idx_x<2>(ixx, d, W, x0, j, k);
          { const F2 v = lds2(psl + 0 * PST); ox0[0] = v.v[0]; ox0[1] = v.v[1]; }
          { const F2 v = lds2(psl + 4 * PST); ox4[0] = v.v[0]; ox4[1] = v.v[1]; }
          { const F2 v = lds2(psl + 6 * PST); ox6[0] = v.v[0]; ox6[1] = v.v[1]; }
        }
        if (ly) {
          psi_idx_row<2>(iyy, (k * (2 * W) + CpmlIdx::slot(j, d.ny, W)) * d.nx + x0, x0, d.nx);
          { const F2 v = lds2(psl + 1 * PST); oy1[0] = v.v[0]; oy1[1] = v.v[1]; }
          { const F2 v = lds2(psl + 3 * PST); oy3[0] = v.v[0]; oy3[1] = v.v[1]; }
          { const F2 v = lds2(psl + 8 * PST); oy8[0] = v.v[0]; oy8[1] = v.v[1]; }
        }
        if (lz) {
          psi_idx_row<2>(izz, (CpmlIdx::slot(gz, d.nz, W) * d.ny + j) * d.nx + x0, x0, d.nx);
          { const F2 v = lds2(psl + 2 * PST); oz2[0] = v.v[0]; oz2[1] = v.v[1]; }
          { const F2 v = lds2(psl + 5 * PST); oz5[0] = v.v[0]; oz5[1] = v.v[1]; }
          { const F2 v = lds2(psl + 7 * PST); oz7[0] = v.v[0]; oz7[1] = v.v[1]; }
        }
      }
      if (lx) {
        float ca[2], cb[2], cah[2], cbh[2];
#pragma unroll
        for (int e = 0; e < 2; ++e) {
          const int c = min(x0 + e, d.nx - 1) - i0;
          ca[e] = ctile.x[0][c]; cb[e] = ctile.x[1][c];
          cah[e] = ctile.x[2][c]; cbh[e] = ctile.x[3][c];
        }
        psi_upd<2>(exx, a.psi[0], ixx, ox0, ca, cb);
        psi_upd<2>(dxvy, a.psi[4], ixx, ox4, cah, cbh);
        psi_upd<2>(dxvz, a.psi[6], ixx, ox6, cah, cbh);
      }
      if (ly) {
        const float ya = ctile.y[0][ty], yb = ctile.y[1][ty];
        const float yah = ctile.y[2][ty], ybh = ctile.y[3][ty];
        const float ca[2] = {ya, ya}, cb[2] = {yb, yb}, cah[2] = {yah, yah}, cbh[2] = {ybh, ybh};
        psi_upd<2>(eyy, a.psi[1], iyy, oy1, ca, cb);
        psi_upd<2>(dyvx, a.psi[3], iyy, oy3, cah, cbh);
        psi_upd<2>(dyvz, a.psi[8], iyy, oy8, cah, cbh);
      }
      if (lz) {
        const float za = __ldg(a.cz.a + gz), zb = __ldg(a.cz.b + gz);
        const float zah = __ldg(a.cz.ah + gz), zbh = __ldg(a.cz.bh + gz);
        const float ca[2] = {za, za}, cb[2] = {zb, zb}, cah[2] = {zah, zah}, cbh[2] = {zbh, zbh};
        psi_upd<2>(ezz, a.psi[2], izz, oz2, ca, cb);
        psi_upd<2>(dzvx, a.psi[5], izz, oz5, cah, cbh);
        psi_upd<2>(dzvy, a.psi[7], izz, oz7, cah, cbh);
      }
      F2 sv[6];
#pragma unroll
      for (int c = 0; c < 6; ++c) sv[c] = lds2(st + L::S + c * L::TS + pt);
      const F2 cl2m = lds2(st + L::C + pt);
      // node w = h/(dt mu) at planes k (wa) and k+1 (wb), rows j (…0) and j+1 (…1), columns
      // x0, x0+1, x0+2; neighbours past the last node clamp to it (O9)
      const float* pa = st + L::WK + ty * RW + 2 * tx;
      const float* pb = st + L::WK1 + ty * RW + 2 * tx;
      const bool ylast = j + 1 >= d.ny, zlast = gz + 1 >= d.nz;
      // (8-byte loads of columns x0 .. x0+3: scalar loads at a 2-float lane stride were 2-way
      // bank conflicts; the column clamp is a register select)
      float wa0[3], wa1[3], wb0[3], wb1[3];
      {
        const F2 a01 = lds2(pa), a23 = lds2(pa + 2), a01n = lds2(pa + RW), a23n = lds2(pa + RW + 2);
        const F2 b01 = lds2(pb), b23 = lds2(pb + 2), b01n = lds2(pb + RW), b23n = lds2(pb + RW + 2);
        const float ra[3] = {a01.v[0], a01.v[1], a23.v[0]}, ran[3] = {a01n.v[0], a01n.v[1], a23n.v[0]};
        const float rb[3] = {b01.v[0], b01.v[1], b23.v[0]}, rbn[3] = {b01n.v[0], b01n.v[1], b23n.v[0]};
        const bool in1 = x0 + 1 < d.nx, in2 = x0 + 2 < d.nx;
#pragma unroll
        for (int c = 0; c < 3; ++c) {
          // column c, clamped to the last node: c if x0 + c < nx, else c - 1 (c = 0 always inside)
          const float va = c == 0 ? ra[0] : c == 1 ? (in1 ? ra[1] : ra[0]) : (in2 ? ra[2] : ra[1]);
          const float van = c == 0 ? ran[0] : c == 1 ? (in1 ? ran[1] : ran[0]) : (in2 ? ran[2] : ran[1]);
          const float vb = c == 0 ? rb[0] : c == 1 ? (in1 ? rb[1] : rb[0]) : (in2 ? rb[2] : rb[1]);
          const float vbn = c == 0 ? rbn[0] : c == 1 ? (in1 ? rbn[1] : rbn[0]) : (in2 ? rbn[2] : rbn[1]);
          wa0[c] = va;
          wa1[c] = ylast ? wa0[c] : van;
          wb0[c] = zlast ? wa0[c] : vb;
          wb1[c] = zlast ? wa1[c] : (ylast ? wb0[c] : vbn);
        }
      }
      const bool surf = a.fs && gz == 0;
      F2 o6[6];
#pragma unroll
      for (int e = 0; e < 2; ++e) {
        // edge mu = harmonic mean of its 4 nodes, 0 if any is 0 (w = inf) (O9); lam = l2m - 2 mu
        const float mxy = 4.0f * rcp_fast((wa0[e] + wa0[e + 1]) + (wa1[e] + wa1[e + 1]));
        const float mxz = 4.0f * rcp_fast((wa0[e] + wa0[e + 1]) + (wb0[e] + wb0[e + 1]));
        const float myz = 4.0f * rcp_fast((wa0[e] + wa1[e]) + (wb0[e] + wb1[e]));
        const float l2m = cl2m.v[e], lam = l2m - 2.0f * rcp_fast(wa0[e]);
        float ez = ezz[e];
        if (surf) ez = -(lam / l2m) * (exx[e] + eyy[e]);  // O16 surface row
        float sxx = sv[0].v[e] + fmaf(l2m, exx[e], lam * (eyy[e] + ez));
        float syy = sv[1].v[e] + fmaf(l2m, eyy[e], lam * (exx[e] + ez));
        float szz = sv[2].v[e] + fmaf(l2m, ez, lam * (exx[e] + eyy[e]));
        if (srel0 - (long long)(k + GZ) * PS == e) {
          const float sa = a.src.get();
          sxx -= sa;
          syy -= sa;
          szz -= sa;
        }
        if (surf) szz = 0.0f;
        o6[0].v[e] = sxx;
        o6[1].v[e] = syy;
        o6[2].v[e] = szz;
        o6[3].v[e] = fmaf(mxy, dyvx[e] + dxvy[e], sv[3].v[e]);
        o6[4].v[e] = fmaf(mxz, dzvx[e] + dxvz[e], sv[4].v[e]);
        o6[5].v[e] = fmaf(myz, dzvy[e] + dyvz[e], sv[5].v[e]);
      }
      // (one x-bound branch for the 6 stores; ghost tests only on boundary planes, as el_v)
      if (x0 + 1 < d.nx) {
#pragma unroll
        for (int c = 0; c < 6; ++c) *reinterpret_cast<float2*>(a.f[ESXX + c] + o) = make_float2(o6[c].v[0], o6[c].v[1]);
      } else {
#pragma unroll
        for (int c = 0; c < 6; ++c) a.f[ESXX + c][o] = o6[c].v[0];
      }
      if (ghk && (k < 4 || k >= d.nzl - 4)) {
        ghost_st2(a.gh[0], o, k, d.nzl, o6[2], x0, d.nx);
        ghost_st2(a.gh[1], o, k, d.nzl, o6[4], x0, d.nx);
        ghost_st2(a.gh[2], o, k, d.nzl, o6[5], x0, d.nx);
      }
      if (SNAP) {
        const long long cix = ((long long)k * d.ny + j) * d.nx + x0;
#pragma unroll
        for (int e = 0; e < 2; ++e)
          if (x0 + e < d.nx) a.snap[cix + e] = -((o6[0].v[e] + o6[1].v[e]) + o6[2].v[e]) / 3.0f;
      }
    }
    if (SEIS_EL_SPSA && W > 0 && it + 1 < np) psi_issue(k + 1);  // (own slots are consumed)
    if (EL_WS) {
      __syncwarp();
      if (tx == 0) mbar_arrive(&ebar[s]);
    } else {
      stage_release<(SEIS_WR_EL != 0)>(&cnt[s], tid, it + EL_SNS < np, [&] {
        issue(s, k + EL_SNS);
        if (L2PF && it + EL_SNS + L2PF < np) issue(s, k + EL_SNS + L2PF, true);
      });
    }
#pragma unroll
    for (int t = 0; t < 7; ++t) {
      qx[t] = qx[t + 1];
      qy[t] = qy[t + 1];
      qz[t] = qz[t + 1];
    }
  }
}

// (region = 3) one launch, the code path chosen per block: blocks whose tile and z-chunk hold
// no C-PML point run the body without the memory-variable code (as the lean instantiation)
template <int BY, bool SNAP, bool CP>
__global__ void __launch_bounds__(NTX2 *(BY + EL_WS), SEIS_EL_MINB > 0 ? SEIS_EL_MINB : (BY <= 8 ? 2 : 1)) el_s_kernel(const __grid_constant__ ElSArgs a) {
  if (CP && a.region == 3) {
    const int k0 = (a.ch0 + (int)blockIdx.z * a.chs) * a.zc;
    const int k1 = min(k0 + a.zc, a.d.nzl);
    if (!el_block_in_layers(a.d, a.W, a.zlo, blockIdx.x * TXE, blockIdx.y * BY, BY, k0, k1)) {
      el_s_body<BY, SNAP, false>(a);
      return;
    }
  }
  el_s_body<BY, SNAP, CP>(a);
}



}  // namespace seis
