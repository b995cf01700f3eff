// kernels_acoustic.cuh — Eq 2 in 3D: variable-density acoustic,
// first-order staggered system, leapfrog (O2, O8), C-PML (O7).
//
//   V:  psi_{p,d} <- bh_d psi_{p,d} + ah_d D+_d p;   q_d += (dt b_d / h)(D+_d p + psi_{p,d})
//   P:  psi_{q,d} <- b_d  psi_{q,d} + a_d  D-_d q_d;  p += (dt K / h) sum_d (D-_d q_d + psi_{q,d})
// with h D+ f_{i+1/2} = sum_m d_m (f_{i+m} - f_{i-m+1}), h D- g_i = sum_m d_m (g_{i+m-1} - g_{i-m})
// (psi is stored multiplied by h, so both updates work on the unscaled differences).
//
// Two z-marching kernels per step, 64 x BY tiles, 4 x-points per
// thread.  V: the p tile (x/y halo 4), the q_x, q_y, q_z tiles, the rho tile
// (+1 in x and y), rho at plane k+1 and p at plane k+4 (the feed of p's float4
// z-queue) arrive by TMA in an NS-deep mbarrier ring; the face buoyancy
// 2/(rho_i + rho_{i+1}) is evaluated on the fly (O8), so V moves 32 B per point.  P: the q_x (x halo) and q_y (y halo) tiles,
// p and dt K/h by TMA, q_z from a register queue.  Fused epilogues: P adds the
// source and stores the snapshot; V applies the imaging
// condition to its input p (O15).
#pragma once
#include "common.cuh"

namespace seis {

struct CpmlAxis {
  const float* __restrict__ a;   // integer nodes
  const float* __restrict__ b;
  const float* __restrict__ ah;  // half nodes i + 1/2
  const float* __restrict__ bh;
};

#ifndef SEIS_AC_NS
#define SEIS_AC_NS 3
#endif
#ifndef SEIS_AC_VNS
#define SEIS_AC_VNS 3
#endif
constexpr int AC_NS = SEIS_AC_NS;    // P kernel ring depth
// launch bounds of the V / P kernels: minimum resident blocks per SM (0 = unspecified)
#ifndef SEIS_AC_MINB
#define SEIS_AC_MINB 0
#endif
#if SEIS_AC_MINB > 0
#define SEIS_AC_LB(n) __launch_bounds__(n, SEIS_AC_MINB)
#else
#define SEIS_AC_LB(n) __launch_bounds__(n)
#endif
constexpr int AC_VNS = SEIS_AC_VNS;  // V kernel ring depth
// L2 prefetch of the C-PML memory variables SEIS_AC_{V,P}PSIPF planes ahead (0 = off), one
// lane per 128-byte slab line: x slab [nzl][ny][2W], y slab [nzl][2W][nx], z slab [2W][ny][nx]
#ifndef SEIS_AC_VPSIPF
#define SEIS_AC_VPSIPF 2  // ac_v 0.759 -> 0.741 ms at C2 (1: 0.745, 3: 0.743, 4: 0.746); ac_p: slower (0.553 vs 0.547), off (profiles/r02_ac_psipf.log)
#endif
#ifndef SEIS_AC_PPSIPF
#define SEIS_AC_PPSIPF 0
#endif
__device__ __forceinline__ void ac_psi_prefetch(const float* px, const float* py, const float* pz, const Dims& d,
                                                int W, int zlo, int tx, int x0, int j, bool lx, bool ly, int kk) {
  if (kk >= d.nzl || (tx & 7) != 0) return;
  if (lx) prefetch_l2(px + (kk * d.ny + j) * (2 * W) + (x0 < W ? 0 : W));
  if (ly) prefetch_l2(py + (kk * (2 * W) + CpmlIdx::slot(j, d.ny, W)) * d.nx + x0);
  const int gz = kk + d.z0;
  if (CpmlIdx::in(gz, d.nz, W, zlo)) prefetch_l2(pz + (CpmlIdx::slot(gz, d.nz, W) * d.ny + j) * d.nx + x0);
}

struct AcVArgs {
  CUtensorMap mp;                 // p tile, box (64+8) x (BY+8) x 1
  CUtensorMap mqx, mqy, mqz;      // q, box 64 x BY x 1
  CUtensorMap mr;                 // rho tile, box (64+4) x (BY+1) x 1 (x+1, y+1 neighbours)
  CUtensorMap mpq;                // p interior (z-queue feed, plane k+4), box 64 x BY x 1
  CUtensorMap mrz;                // rho interior (z faces, plane k+1), box 64 x BY x 1
  const float* __restrict__ p;
  const float* __restrict__ rho;  // density (padded; z ghosts filled from the neighbour slabs)
  float dth;                      // dt / h
  float* __restrict__ qx;
  float* __restrict__ qy;
  float* __restrict__ qz;
  int W;                          // C-PML slab width per face (nb + 1), 0 = no layer
  int zlo;                        // 1 if the top z face has a layer
  CpmlAxis cx, cy, cz;
  float* __restrict__ psx;        // psi_{p,x} [nzl][ny][2W]
  float* __restrict__ psy;        // psi_{p,y} [nzl][2W][nx]
  float* __restrict__ psz;        // psi_{p,z} [2W][ny][nx] (global z slots)
  Dims d;
  int zc;
  int ch0, chs;                  // z-chunk of blockIdx.z = ch0 + blockIdx.z * chs (boundary / interior split)
  const float* __restrict__ imgS; // imaging: img += S * p (input level), or nullptr
  SnapRef imgR;                   // the same (fp32 or 24-bit), what the IMG kernel reads
  float* __restrict__ img;
  Ghost gh;                       // direct ghost stores of q_z (f4)
};

template <int BY>
struct AcVStage {
  static constexpr int W = TXV + 8, T = TXV * BY, RW = TXV + 4;
  static constexpr int P = 0, QX = (BY + 8) * W, QY = QX + T, QZ = QY + T, PQ = QZ + T, RZ = PQ + T,
                       R = RZ + T, SIZE = R + ((RW * (BY + 1) + 31) / 32) * 32;
  static constexpr uint32_t BYTES = ((BY + 8) * W + 5 * T + RW * (BY + 1)) * 4;
  static constexpr size_t smem_bytes() { return (size_t)AC_VNS * SIZE * 4 + 128; }
};

template <int BY, bool IMG>
__global__ void SEIS_AC_LB(NTX * BY) ac_v_kernel(const __grid_constant__ AcVArgs a) {
  using L = AcVStage<BY>;
  constexpr int W = L::W, RW = L::RW;
  constexpr uint32_t TX_BYTES = L::BYTES;
  extern __shared__ __align__(128) float sm_raw[];
  float* sm = align128(sm_raw);
  __shared__ __align__(8) uint64_t bar[AC_VNS];
  __shared__ uint32_t cnt[AC_VNS];
  const Dims& d = a.d;
  const int tx = threadIdx.x, ty = threadIdx.y, tid = ty * NTX + tx;
  const int i0 = blockIdx.x * TXV, j0 = blockIdx.y * BY;
  const int x0 = i0 + 4 * tx, j = j0 + ty;
  const int k0 = (a.ch0 + (int)blockIdx.z * a.chs) * a.zc;
  const int k1 = min(k0 + a.zc, d.nzl);
  const int np = k1 - k0;
  const bool own = (x0 < d.nx) && (j < d.ny);
  const long long PS = d.PS;
  const long long oc = (long long)(j + G) * d.PX + (x0 + G);
  const float* __restrict__ p = a.p;
  const int Wl = a.W;
  const bool lx = Wl > 0 && (x0 < Wl || x0 + 3 >= d.nx - Wl);  // some component may be in the x layer
  const bool ly = Wl > 0 && CpmlIdx::in(j, d.ny, Wl, true);
  auto issue = [&](int s, int k, bool pf = false) {
    float* st = sm + s * L::SIZE;
    const int z = k + GZ, x = i0 + G, y = j0 + G;
    if (!pf) mbar_expect_tx(&bar[s], TX_BYTES);
    tma_ld(pf, st + L::P, &a.mp, &bar[s], i0, j0, z);
    tma_ld(pf, st + L::QX, &a.mqx, &bar[s], x, y, z);
    tma_ld(pf, st + L::QY, &a.mqy, &bar[s], x, y, z);
    tma_ld(pf, st + L::QZ, &a.mqz, &bar[s], x, y, z);
    tma_ld(pf, st + L::R, &a.mr, &bar[s], x, y, z);
    tma_ld(pf, st + L::PQ, &a.mpq, &bar[s], x, y, z + 4);
    tma_ld(pf, st + L::RZ, &a.mrz, &bar[s], x, y, z + 1);
  };
  if (tid == 0) {
    for (int s = 0; s < AC_VNS; ++s) {
      mbar_init(&bar[s], 1);
      cnt[s] = 0u;
    }
    mbar_fence_init();
  }
  __syncthreads();
  if (tid == 0)
    for (int s = 0; s < AC_VNS && s < np; ++s) issue(s, k0 + s);
  if (tid == 0)
    for (int t = 0; t < L2PF && AC_VNS + t < np; ++t) issue(0, k0 + AC_VNS + t, true);
  F4 r[8];  // p at k-3 .. k+4; plane k+4 arrives with stage k (TMA)
#pragma unroll
  for (int t = 0; t < 7; ++t) r[t] = ldg4(p + (long long)(k0 - 3 + t + GZ) * PS + oc);
  const float dth = a.dth;

  const bool ghk = a.gh.lo || a.gh.hi;  // does this slab store a neighbour's ghost planes (f4)?
  SEIS_UNROLL(SEIS_ZU_AC)
  for (int it = 0; it < np; ++it) {
    const int k = k0 + it;
    const int s = it % AC_VNS;
    const long long o = (long long)(k + GZ) * PS + oc;
    // C-PML: old psi values are loaded before the wait (latency overlap)
    const int gz = k + d.z0;
    const bool lz = Wl > 0 && CpmlIdx::in(gz, d.nz, Wl, a.zlo);
    int ixx[4], iyy[4], izz[4];  // 32-bit compact-slab indices (fewer live registers)
    float ox[4], oy[4], oz[4];
    if (own && lx) {
      psi_idx_x<4>(ixx, d, Wl, x0, j, k);
      psi_ld<4>(ox, a.psx, ixx);
    }
    if (own && ly) {
      psi_idx_row<4>(iyy, (k * (2 * Wl) + CpmlIdx::slot(j, d.ny, Wl)) * d.nx + x0, x0, d.nx);
      psi_ld<4>(oy, a.psy, iyy);
    }
    if (own && lz) {
      psi_idx_row<4>(izz, (CpmlIdx::slot(gz, d.nz, Wl) * d.ny + j) * d.nx + x0, x0, d.nx);
      psi_ld<4>(oz, a.psz, izz);
    }
    if (SEIS_AC_VPSIPF > 0 && Wl > 0 && own)
      ac_psi_prefetch(a.psx, a.psy, a.psz, d, Wl, a.zlo, tx, x0, j, lx, ly, k + SEIS_AC_VPSIPF);
    mbar_wait(&bar[s], (it / AC_VNS) & 1);
    const float* st = sm + s * L::SIZE;
    r[7] = lds4(st + L::PQ + ty * TXV + 4 * tx);
    const F4 rz1 = lds4(st + L::RZ + ty * TXV + 4 * tx);  // rho(k+1)
    const float* c = st + L::P + (ty + 4) * W + 4 * tx + 4;  // p(x0, j, k)
    float xv[12];                                             // p(x0-4 .. x0+7, j)
    {
      const F4 a0 = lds4(c - 4), a1 = lds4(c), a2 = lds4(c + 4);
#pragma unroll
      for (int e = 0; e < 4; ++e) {
        xv[e] = a0.v[e];
        xv[4 + e] = a1.v[e];
        xv[8 + e] = a2.v[e];
      }
    }
    F4 yr[8];  // p rows j-3 .. j+4
#pragma unroll
    for (int m = 0; m < 8; ++m) yr[m] = (m == 3) ? F4{{xv[4], xv[5], xv[6], xv[7]}} : lds4(c + (m - 3) * W);
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
    if (own) {
      if (lx) {
        float ca[4], cb[4];
#pragma unroll
        for (int e = 0; e < 4; ++e) {
          const int x = min(x0 + e, d.nx - 1);
          ca[e] = __ldg(a.cx.ah + x);
          cb[e] = __ldg(a.cx.bh + x);
        }
        psi_upd<4>(dx, a.psx, ixx, ox, ca, cb);
      }
      if (ly) {
        const float ya = __ldg(a.cy.ah + j), yb = __ldg(a.cy.bh + j);
        const float ca[4] = {ya, ya, ya, ya}, cb[4] = {yb, yb, yb, yb};
        psi_upd<4>(dy, a.psy, iyy, oy, ca, cb);
      }
      if (lz) {
        const float za = __ldg(a.cz.ah + gz), zb = __ldg(a.cz.bh + gz);
        const float ca[4] = {za, za, za, za}, cb[4] = {zb, zb, zb, zb};
        psi_upd<4>(dz, a.psz, izz, oz, ca, cb);
      }
      const int pt = ty * TXV + 4 * tx;
      const F4 qxo = lds4(st + L::QX + pt), qyo = lds4(st + L::QY + pt), qzo = lds4(st + L::QZ + pt);
      // face buoyancy dt b/h = (dt/h) 2 / (rho_i + rho_{i+1}), last face clamps (O8)
      const float* rc = st + L::R + ty * RW + 4 * tx;
      const F4 r0 = lds4(rc), rxn = lds4(rc + 4), ryn = lds4(rc + RW);
      const float rx5 = rxn.v[0];
      const bool zlast = gz + 1 >= d.nz;
      F4 ox, oy, oz;
#pragma unroll
      for (int e = 0; e < 4; ++e) {
        const float rxp = (x0 + e + 1 < d.nx) ? (e < 3 ? r0.v[e + 1] : rx5) : r0.v[e];
        const float ryp = (j + 1 < d.ny) ? ryn.v[e] : r0.v[e];
        const float rzp = zlast ? r0.v[e] : rz1.v[e];
        const float bx = dth * (2.0f * rcp_fast(r0.v[e] + rxp));
        const float by = dth * (2.0f * rcp_fast(r0.v[e] + ryp));
        const float bz = dth * (2.0f * rcp_fast(r0.v[e] + rzp));
        ox.v[e] = fmaf(bx, dx[e], qxo.v[e]);
        oy.v[e] = fmaf(by, dy[e], qyo.v[e]);
        oz.v[e] = fmaf(bz, dz[e], qzo.v[e]);
      }
      // one x-bound branch for the 3 stores; ghost tests only on a slab's 4 boundary planes
      if (x0 + 3 < d.nx) {
        st4(a.qx + o, ox);
        st4(a.qy + o, oy);
        st4(a.qz + o, oz);
      } else {
        st4_masked(a.qx + o, ox, x0, d.nx, false);
        st4_masked(a.qy + o, oy, x0, d.nx, false);
        st4_masked(a.qz + o, oz, x0, d.nx, false);
      }
      if (ghk && (k < 4 || k >= d.nzl - 4)) ghost_st4(a.gh, o, k, d.nzl, oz, x0, d.nx);
      if (IMG) {
        const long long cix = ((long long)k * d.ny + j) * d.nx + x0;
        F4 im;
#pragma unroll
        for (int e = 0; e < 4; ++e)
          im.v[e] = (x0 + e < d.nx) ? fmaf(a.imgR.at(cix + e), r[3].v[e], a.img[cix + e]) : 0.f;
        st4_masked(a.img + cix, im, x0, d.nx, false);
      }
    }
    stage_release(&cnt[s], tid, it + AC_VNS < np, [&] {
      issue(s, k + AC_VNS);
      if (L2PF && it + AC_VNS + L2PF < np) issue(s, k + AC_VNS + L2PF, true);
    });
#pragma unroll
    for (int t = 0; t < 7; ++t) r[t] = r[t + 1];
  }
}

struct AcPArgs {
  CUtensorMap mqx;                // q_x, box (64+8) x BY x 1
  CUtensorMap mqy;                // q_y, box 64 x (BY+8) x 1
  CUtensorMap mpp;                // p, box 64 x BY x 1
  CUtensorMap mk;                 // dt K / h, box 64 x BY x 1
  CUtensorMap mqq;                // q_z interior (z-queue feed, plane k+3), box 64 x BY x 1
  float* __restrict__ p;
  const float* __restrict__ qz;
  int W;
  int zlo;
  CpmlAxis cx, cy, cz;
  float* __restrict__ pqx;        // psi_{q,x} [nzl][ny][2W]
  float* __restrict__ pqy;        // psi_{q,y} [nzl][2W][nx]
  float* __restrict__ pqz;        // psi_{q,z} [2W][ny][nx]
  Dims d;
  int zc;
  int ch0, chs;                  // z-chunk of blockIdx.z = ch0 + blockIdx.z * chs (boundary / interior split)
  long long src_o;                // padded index of the source in this slab, -1 = none
  SrcAmp src;                     // dt K_s / h^3 * s[n]
  float* __restrict__ snap;       // compact snapshot target, or nullptr
  Ghost gh;                       // direct ghost stores of p (f4)
};

template <int BY>
struct AcPStage {
  static constexpr int WX = TXV + 8, T = TXV * BY;
  static constexpr int QX = 0, QY = BY * WX, P = QY + (BY + 8) * TXV, K = P + T, QQ = K + T, SIZE = QQ + T;
  static constexpr size_t smem_bytes() { return (size_t)AC_NS * SIZE * 4 + 128; }
};

template <int BY, bool SNAP>
__global__ void SEIS_AC_LB(NTX * BY) ac_p_kernel(const __grid_constant__ AcPArgs a) {
  using L = AcPStage<BY>;
  constexpr int WX = L::WX;
  constexpr uint32_t TX_BYTES = L::SIZE * 4;
  extern __shared__ __align__(128) float sm_raw[];
  float* sm = align128(sm_raw);
  __shared__ __align__(8) uint64_t bar[AC_NS];
  __shared__ uint32_t cnt[AC_NS];
  const Dims& d = a.d;
  const int tx = threadIdx.x, ty = threadIdx.y, tid = ty * NTX + tx;
  const int i0 = blockIdx.x * TXV, j0 = blockIdx.y * BY;
  const int x0 = i0 + 4 * tx, j = j0 + ty;
  const int k0 = (a.ch0 + (int)blockIdx.z * a.chs) * a.zc;
  const int k1 = min(k0 + a.zc, d.nzl);
  const int np = k1 - k0;
  const bool own = (x0 < d.nx) && (j < d.ny);
  const long long PS = d.PS;
  const long long oc = (long long)(j + G) * d.PX + (x0 + G);
  const float* __restrict__ qz = a.qz;
  const int Wl = a.W;
  const bool lx = Wl > 0 && (x0 < Wl || x0 + 3 >= d.nx - Wl);
  const bool ly = Wl > 0 && CpmlIdx::in(j, d.ny, Wl, true);
  const bool vec4 = (d.nx & 3) == 0 && x0 + 3 < d.nx;  // (y / z slab groups: one 16-byte access; in ac_p
  // 0.5475 -> 0.545 ms at C2, in ac_v / el_v / el_s slower: profiles/r02_psi_vec_ab.log)
  auto issue = [&](int s, int k, bool pf = false) {
    float* st = sm + s * L::SIZE;
    const int z = k + GZ;
    if (!pf) mbar_expect_tx(&bar[s], TX_BYTES);
    tma_ld(pf, st + L::QX, &a.mqx, &bar[s], i0, j0 + G, z);
    tma_ld(pf, st + L::QY, &a.mqy, &bar[s], i0 + G, j0, z);
    tma_ld(pf, st + L::P, &a.mpp, &bar[s], i0 + G, j0 + G, z);
    tma_ld(pf, st + L::K, &a.mk, &bar[s], i0 + G, j0 + G, z);
    tma_ld(pf, st + L::QQ, &a.mqq, &bar[s], i0 + G, j0 + G, z + 3);
  };
  if (tid == 0) {
    for (int s = 0; s < AC_NS; ++s) {
      mbar_init(&bar[s], 1);
      cnt[s] = 0u;
    }
    mbar_fence_init();
  }
  __syncthreads();
  if (tid == 0)
    for (int s = 0; s < AC_NS && s < np; ++s) issue(s, k0 + s);
  if (tid == 0)
    for (int t = 0; t < L2PF && AC_NS + t < np; ++t) issue(0, k0 + AC_NS + t, true);
  F4 q[8];  // q_z at k-4 .. k+3; plane k+3 arrives with stage k (TMA)
#pragma unroll
  for (int t = 0; t < 7; ++t) q[t] = ldg4(qz + (long long)(k0 - 4 + t + GZ) * PS + oc);
  const SrcHit sh = src_hit(a.src_o, oc, PS, 4);

  const bool ghk = a.gh.lo || a.gh.hi;  // does this slab store a neighbour's ghost planes (f4)?
  int s_ = 0;
  uint32_t ph_ = 0u;
  long long o_ = (long long)(k0 + GZ) * PS + oc;
  SEIS_UNROLL(SEIS_ZU_AC)
  for (int it = 0; it < np; ++it) {
    const int k = k0 + it;
    // ring slot, its phase and the plane offset carried across iterations (no division by the
    // ring depth or 64-bit multiply per plane)
    const int s = s_;
    const uint32_t ph = ph_;
    const long long o = o_;
    o_ += PS;
    if (++s_ == AC_NS) {
      s_ = 0;
      ph_ ^= 1u;
    }
    // C-PML: old psi values are loaded before the wait (latency overlap)
    const int gz = k + d.z0;
    const bool lz = Wl > 0 && CpmlIdx::in(gz, d.nz, Wl, a.zlo);
    int ixx[4], iyy[4], izz[4];  // 32-bit compact-slab indices (fewer live registers)
    float ox[4], oy[4], oz[4];
    if (own && lx) {
      psi_idx_x<4>(ixx, d, Wl, x0, j, k);
      psi_ld<4>(ox, a.pqx, ixx);
    }
    if (own && ly) {
      psi_idx_row<4>(iyy, (k * (2 * Wl) + CpmlIdx::slot(j, d.ny, Wl)) * d.nx + x0, x0, d.nx);
      psi_ld_row<4>(oy, a.pqy, iyy, vec4);
    }
    if (own && lz) {
      psi_idx_row<4>(izz, (CpmlIdx::slot(gz, d.nz, Wl) * d.ny + j) * d.nx + x0, x0, d.nx);
      psi_ld_row<4>(oz, a.pqz, izz, vec4);
    }
    if (SEIS_AC_PPSIPF > 0 && Wl > 0 && own)
      ac_psi_prefetch(a.pqx, a.pqy, a.pqz, d, Wl, a.zlo, tx, x0, j, lx, ly, k + SEIS_AC_PPSIPF);
    mbar_wait(&bar[s], ph);
    const float* st = sm + s * L::SIZE;
    q[7] = lds4(st + L::QQ + ty * TXV + 4 * tx);
    const float* cx = st + L::QX + ty * WX + 4 * tx + 4;      // q_x(x0, j)
    const float* cy = st + L::QY + (ty + 4) * TXV + 4 * tx;   // q_y(x0, j)
    float xv[12];                                             // q_x(x0-4 .. x0+7)
    {
      const F4 a0 = lds4(cx - 4), a1 = lds4(cx), a2 = lds4(cx + 4);
#pragma unroll
      for (int e = 0; e < 4; ++e) {
        xv[e] = a0.v[e];
        xv[4 + e] = a1.v[e];
        xv[8 + e] = a2.v[e];
      }
    }
    F4 yr[8];  // q_y rows j-4 .. j+3
#pragma unroll
    for (int m = 0; m < 8; ++m) yr[m] = lds4(cy + (m - 4) * TXV);
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
      t = SEIS_D1 * (q[4].v[e] - q[3].v[e]);
      t = fmaf(SEIS_D2, q[5].v[e] - q[2].v[e], t);
      t = fmaf(SEIS_D3, q[6].v[e] - q[1].v[e], t);
      dz[e] = fmaf(SEIS_D4, q[7].v[e] - q[0].v[e], t);
    }
    if (own) {
      if (lx) {
        float ca[4], cb[4];
#pragma unroll
        for (int e = 0; e < 4; ++e) {
          const int x = min(x0 + e, d.nx - 1);
          ca[e] = __ldg(a.cx.a + x);
          cb[e] = __ldg(a.cx.b + x);
        }
        psi_upd<4>(dx, a.pqx, ixx, ox, ca, cb);
      }
      if (ly) {
        const float ya = __ldg(a.cy.a + j), yb = __ldg(a.cy.b + j);
        const float ca[4] = {ya, ya, ya, ya}, cb[4] = {yb, yb, yb, yb};
        psi_upd_row<4>(dy, a.pqy, iyy, oy, ca, cb, vec4);
      }
      if (lz) {
        const float za = __ldg(a.cz.a + gz), zb = __ldg(a.cz.b + gz);
        const float ca[4] = {za, za, za, za}, cb[4] = {zb, zb, zb, zb};
        psi_upd_row<4>(dz, a.pqz, izz, oz, ca, cb, vec4);
      }
      const int pt = ty * TXV + 4 * tx;
      const F4 pv = lds4(st + L::P + pt), kv = lds4(st + L::K + pt);
      F4 out;
#pragma unroll
      for (int e = 0; e < 4; ++e) out.v[e] = fmaf(kv.v[e], (dx[e] + dy[e]) + dz[e], pv.v[e]);
      if (sh.at(k)) {  // (selects: a branch per component became a local-memory array)
        const float sa = a.src.get();
        const int se = sh.e();
#pragma unroll
        for (int e = 0; e < 4; ++e) out.v[e] = (se == e) ? out.v[e] + sa : out.v[e];
      }
      st4_masked(a.p + o, out, x0, d.nx, true);
      if (ghk && (k < 4 || k >= d.nzl - 4)) ghost_st4(a.gh, o, k, d.nzl, out, x0, d.nx);
      if (SNAP) st4_masked(a.snap + ((long long)k * d.ny + j) * d.nx + x0, out, x0, d.nx, (d.nx & 3) == 0);
    }
    stage_release(&cnt[s], tid, it + AC_NS < np, [&] {
      issue(s, k + AC_NS);
      if (L2PF && it + AC_NS + L2PF < np) issue(s, k + AC_NS + L2PF, true);
    });
#pragma unroll
    for (int t = 0; t < 7; ++t) q[t] = q[t + 1];
  }
}

}  // namespace seis
