// kernels_acoustic.cuh — Eq 2 in 3D: variable-density acoustic,
// first-order staggered system, leapfrog (O2, O8), C-PML (O7).
//
//   V:  psi_{p,d} <- bh_d psi_{p,d} + ah_d D+_d p;   q_d += (dt b_d / h)(D+_d p + psi_{p,d})
//   P:  psi_{q,d} <- b_d  psi_{q,d} + a_d  D-_d q_d;  p += (dt K / h) sum_d (D-_d q_d + psi_{q,d})
// with h D+ f_{i+1/2} = sum_m d_m (f_{i+m} - f_{i-m+1}), h D- g_i = sum_m d_m (g_{i+m-1} - g_{i-m})
// (psi is stored multiplied by h, so both updates work on the unscaled differences).
//
// Two z-marching kernels per step.  V: p plane tile (x/y halo 4)
// by TMA through an NS-stage mbarrier ring, p's z-neighbours from a register
// queue, q_x, q_y, q_z and the face buoyancies dt b/h as coalesced streams
// prefetched one plane ahead.  P: q_x (x halo) and q_y (y halo) tiles by TMA,
// q_z from a register queue, p and dt K/h streamed.  Fused epilogues: P adds the
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

constexpr int AC_NS = 4;

struct AcVArgs {
  CUtensorMap mp;                 // p, box (32+8) x (BY+8) x 1
  const float* __restrict__ p;
  float* __restrict__ qx;
  float* __restrict__ qy;
  float* __restrict__ qz;
  const float* __restrict__ bx;  // dt * 2/(rho_i + rho_{i+1}) / h on x faces (padded)
  const float* __restrict__ by;
  const float* __restrict__ bz;
  int W;                          // C-PML slab width per face (nb + 1), 0 = no layer
  int zlo;                        // 1 if the top z face has a layer
  CpmlAxis cx, cy, cz;
  float* __restrict__ psx;        // psi_{p,x} [nzl][ny][2W]
  float* __restrict__ psy;        // psi_{p,y} [nzl][2W][nx]
  float* __restrict__ psz;        // psi_{p,z} [2W][ny][nx] (global z slots)
  Dims d;
  int zc;
  const float* __restrict__ imgS; // imaging: img += S * p (input level), or nullptr
  float* __restrict__ img;
};

template <int BY, bool IMG>
__global__ void __launch_bounds__(TXW * BY) ac_v_kernel(const __grid_constant__ AcVArgs a) {
  constexpr int W = TXW + 8;
  constexpr int TILE = (BY + 8) * W;
  constexpr uint32_t TX_BYTES = TILE * 4;
  __shared__ __align__(128) float sm[AC_NS * TILE];
  __shared__ __align__(8) uint64_t bar[AC_NS];
  const Dims& d = a.d;
  const int tx = threadIdx.x, ty = threadIdx.y, tid = ty * TXW + tx;
  const int i0 = blockIdx.x * TXW, j0 = blockIdx.y * BY;
  const int i = i0 + tx, j = j0 + ty;
  const int k0 = blockIdx.z * a.zc;
  const int k1 = min(k0 + a.zc, d.nzl);
  const int np = k1 - k0;
  const bool own = (i < d.nx) && (j < d.ny);
  const long long PS = d.PS;
  const long long oc = (long long)(j + G) * d.PX + (i + G);
  const float* __restrict__ p = a.p;
  const int Wl = a.W;
  const bool lx = Wl > 0 && CpmlIdx::in(i, d.nx, Wl, true);
  const bool ly = Wl > 0 && CpmlIdx::in(j, d.ny, Wl, true);

  if (tid == 0) {
    for (int s = 0; s < AC_NS; ++s) mbar_init(&bar[s], 1);
    mbar_fence_init();
  }
  __syncthreads();
  if (tid == 0) {
    for (int s = 0; s < AC_NS && s < np; ++s) {
      mbar_expect_tx(&bar[s], TX_BYTES);
      tma_load_3d(sm + s * TILE, &a.mp, &bar[s], i0, j0, k0 + s + G);
    }
  }
  float r0, r1, r2, r3, r4, r5, r6, r7;  // p at k-3 .. k+4
  r0 = __ldg(p + (long long)(k0 - 3 + G) * PS + oc);
  r1 = __ldg(p + (long long)(k0 - 2 + G) * PS + oc);
  r2 = __ldg(p + (long long)(k0 - 1 + G) * PS + oc);
  r3 = __ldg(p + (long long)(k0 + G) * PS + oc);
  r4 = __ldg(p + (long long)(k0 + 1 + G) * PS + oc);
  r5 = __ldg(p + (long long)(k0 + 2 + G) * PS + oc);
  r6 = __ldg(p + (long long)(k0 + 3 + G) * PS + oc);
  float r7n = __ldg(p + (long long)(k0 + 4 + G) * PS + oc);
  float qxn = 0.f, qyn = 0.f, qzn = 0.f, bxn = 0.f, byn = 0.f, bzn = 0.f;
  if (own && np > 0) {
    const long long o = (long long)(k0 + G) * PS + oc;
    qxn = a.qx[o]; qyn = a.qy[o]; qzn = a.qz[o];
    bxn = __ldg(a.bx + o); byn = __ldg(a.by + o); bzn = __ldg(a.bz + o);
  }

  for (int it = 0; it < np; ++it) {
    const int k = k0 + it;
    const int s = it % AC_NS;
    const long long o = (long long)(k + G) * PS + oc;
    r7 = r7n;
    const float qxv = qxn, qyv = qyn, qzv = qzn, bxv = bxn, byv = byn, bzv = bzn;
    if (it + 1 < np) {
      r7n = __ldg(p + o + 5 * PS);
      if (own) {
        qxn = a.qx[o + PS]; qyn = a.qy[o + PS]; qzn = a.qz[o + PS];
        bxn = __ldg(a.bx + o + PS); byn = __ldg(a.by + o + PS); bzn = __ldg(a.bz + o + PS);
      }
    }
    mbar_wait(&bar[s], (it / AC_NS) & 1);
    const float* c = sm + s * TILE + (ty + 4) * W + tx + 4;
    float dx = SEIS_D1 * (c[1] - c[0]);
    dx = fmaf(SEIS_D2, c[2] - c[-1], dx);
    dx = fmaf(SEIS_D3, c[3] - c[-2], dx);
    dx = fmaf(SEIS_D4, c[4] - c[-3], dx);
    float dy = SEIS_D1 * (c[W] - c[0]);
    dy = fmaf(SEIS_D2, c[2 * W] - c[-W], dy);
    dy = fmaf(SEIS_D3, c[3 * W] - c[-2 * W], dy);
    dy = fmaf(SEIS_D4, c[4 * W] - c[-3 * W], dy);
    float dz = SEIS_D1 * (r4 - r3);
    dz = fmaf(SEIS_D2, r5 - r2, dz);
    dz = fmaf(SEIS_D3, r6 - r1, dz);
    dz = fmaf(SEIS_D4, r7 - r0, dz);
    if (own) {
      if (Wl > 0) {
        if (lx) {
          const long long ix = ((long long)k * d.ny + j) * (2 * Wl) + CpmlIdx::slot(i, d.nx, Wl);
          const float ps = fmaf(__ldg(a.cx.bh + i), a.psx[ix], __ldg(a.cx.ah + i) * dx);
          a.psx[ix] = ps;
          dx += ps;
        }
        if (ly) {
          const long long iy = ((long long)k * (2 * Wl) + CpmlIdx::slot(j, d.ny, Wl)) * d.nx + i;
          const float ps = fmaf(__ldg(a.cy.bh + j), a.psy[iy], __ldg(a.cy.ah + j) * dy);
          a.psy[iy] = ps;
          dy += ps;
        }
        const int gz = k + d.z0;
        if (CpmlIdx::in(gz, d.nz, Wl, a.zlo)) {
          const long long iz = ((long long)CpmlIdx::slot(gz, d.nz, Wl) * d.ny + j) * d.nx + i;
          const float ps = fmaf(__ldg(a.cz.bh + gz), a.psz[iz], __ldg(a.cz.ah + gz) * dz);
          a.psz[iz] = ps;
          dz += ps;
        }
      }
      a.qx[o] = fmaf(bxv, dx, qxv);
      a.qy[o] = fmaf(byv, dy, qyv);
      a.qz[o] = fmaf(bzv, dz, qzv);
      if (IMG) {
        const long long cix = ((long long)k * d.ny + j) * d.nx + i;
        a.img[cix] = fmaf(__ldg(a.imgS + cix), r3, a.img[cix]);
      }
    }
    __syncthreads();
    if (tid == 0 && it + AC_NS < np) {
      fence_proxy_async();
      mbar_expect_tx(&bar[s], TX_BYTES);
      tma_load_3d(sm + s * TILE, &a.mp, &bar[s], i0, j0, k + AC_NS + G);
    }
    r0 = r1; r1 = r2; r2 = r3; r3 = r4; r4 = r5; r5 = r6; r6 = r7;
  }
}

struct AcPArgs {
  CUtensorMap mqx;                // q_x, box (32+8) x BY x 1
  CUtensorMap mqy;                // q_y, box 32 x (BY+8) x 1
  float* __restrict__ p;
  const float* __restrict__ qz;
  const float* __restrict__ kdt;  // dt * rho v^2 / h (padded)
  int W;
  int zlo;
  CpmlAxis cx, cy, cz;
  float* __restrict__ pqx;        // psi_{q,x} [nzl][ny][2W]
  float* __restrict__ pqy;        // psi_{q,y} [nzl][2W][nx]
  float* __restrict__ pqz;        // psi_{q,z} [2W][ny][nx]
  Dims d;
  int zc;
  long long src_o;                // padded index of the source in this slab, -1 = none
  float src_amp;                  // dt K_s / h^3 * s[n]
  float* __restrict__ snap;       // compact snapshot target, or nullptr
};

template <int BY, bool SNAP>
__global__ void __launch_bounds__(TXW * BY) ac_p_kernel(const __grid_constant__ AcPArgs a) {
  constexpr int WX = TXW + 8;
  constexpr int TQX = BY * WX;           // q_x tile (x halo)
  constexpr int TQY = (BY + 8) * TXW;    // q_y tile (y halo)
  constexpr int STAGE = TQX + TQY;       // both multiples of 32 floats (128 B)
  constexpr uint32_t TX_BYTES = STAGE * 4;
  __shared__ __align__(128) float sm[AC_NS * STAGE];
  __shared__ __align__(8) uint64_t bar[AC_NS];
  const Dims& d = a.d;
  const int tx = threadIdx.x, ty = threadIdx.y, tid = ty * TXW + tx;
  const int i0 = blockIdx.x * TXW, j0 = blockIdx.y * BY;
  const int i = i0 + tx, j = j0 + ty;
  const int k0 = blockIdx.z * a.zc;
  const int k1 = min(k0 + a.zc, d.nzl);
  const int np = k1 - k0;
  const bool own = (i < d.nx) && (j < d.ny);
  const long long PS = d.PS;
  const long long oc = (long long)(j + G) * d.PX + (i + G);
  const float* __restrict__ qz = a.qz;
  const int Wl = a.W;
  const bool lx = Wl > 0 && CpmlIdx::in(i, d.nx, Wl, true);
  const bool ly = Wl > 0 && CpmlIdx::in(j, d.ny, Wl, true);

  if (tid == 0) {
    for (int s = 0; s < AC_NS; ++s) mbar_init(&bar[s], 1);
    mbar_fence_init();
  }
  __syncthreads();
  if (tid == 0) {
    for (int s = 0; s < AC_NS && s < np; ++s) {
      mbar_expect_tx(&bar[s], TX_BYTES);
      tma_load_3d(sm + s * STAGE, &a.mqx, &bar[s], i0, j0 + G, k0 + s + G);
      tma_load_3d(sm + s * STAGE + TQX, &a.mqy, &bar[s], i0 + G, j0, k0 + s + G);
    }
  }
  float s0, s1, s2, s3, s4, s5, s6, s7;  // q_z at k-4 .. k+3
  s0 = __ldg(qz + (long long)(k0 - 4 + G) * PS + oc);
  s1 = __ldg(qz + (long long)(k0 - 3 + G) * PS + oc);
  s2 = __ldg(qz + (long long)(k0 - 2 + G) * PS + oc);
  s3 = __ldg(qz + (long long)(k0 - 1 + G) * PS + oc);
  s4 = __ldg(qz + (long long)(k0 + G) * PS + oc);
  s5 = __ldg(qz + (long long)(k0 + 1 + G) * PS + oc);
  s6 = __ldg(qz + (long long)(k0 + 2 + G) * PS + oc);
  float s7n = __ldg(qz + (long long)(k0 + 3 + G) * PS + oc);
  float pn = 0.f, kn = 0.f;
  if (own && np > 0) {
    const long long o = (long long)(k0 + G) * PS + oc;
    pn = a.p[o];
    kn = __ldg(a.kdt + o);
  }

  for (int it = 0; it < np; ++it) {
    const int k = k0 + it;
    const int s = it % AC_NS;
    const long long o = (long long)(k + G) * PS + oc;
    s7 = s7n;
    const float pv = pn, kv = kn;
    if (it + 1 < np) {
      s7n = __ldg(qz + o + 4 * PS);
      if (own) {
        pn = a.p[o + PS];
        kn = __ldg(a.kdt + o + PS);
      }
    }
    mbar_wait(&bar[s], (it / AC_NS) & 1);
    const float* cx = sm + s * STAGE + ty * WX + tx + 4;
    const float* cy = sm + s * STAGE + TQX + (ty + 4) * TXW + tx;
    float dx = SEIS_D1 * (cx[0] - cx[-1]);
    dx = fmaf(SEIS_D2, cx[1] - cx[-2], dx);
    dx = fmaf(SEIS_D3, cx[2] - cx[-3], dx);
    dx = fmaf(SEIS_D4, cx[3] - cx[-4], dx);
    float dy = SEIS_D1 * (cy[0] - cy[-TXW]);
    dy = fmaf(SEIS_D2, cy[TXW] - cy[-2 * TXW], dy);
    dy = fmaf(SEIS_D3, cy[2 * TXW] - cy[-3 * TXW], dy);
    dy = fmaf(SEIS_D4, cy[3 * TXW] - cy[-4 * TXW], dy);
    float dz = SEIS_D1 * (s4 - s3);
    dz = fmaf(SEIS_D2, s5 - s2, dz);
    dz = fmaf(SEIS_D3, s6 - s1, dz);
    dz = fmaf(SEIS_D4, s7 - s0, dz);
    if (own) {
      if (Wl > 0) {
        if (lx) {
          const long long ix = ((long long)k * d.ny + j) * (2 * Wl) + CpmlIdx::slot(i, d.nx, Wl);
          const float ps = fmaf(__ldg(a.cx.b + i), a.pqx[ix], __ldg(a.cx.a + i) * dx);
          a.pqx[ix] = ps;
          dx += ps;
        }
        if (ly) {
          const long long iy = ((long long)k * (2 * Wl) + CpmlIdx::slot(j, d.ny, Wl)) * d.nx + i;
          const float ps = fmaf(__ldg(a.cy.b + j), a.pqy[iy], __ldg(a.cy.a + j) * dy);
          a.pqy[iy] = ps;
          dy += ps;
        }
        const int gz = k + d.z0;
        if (CpmlIdx::in(gz, d.nz, Wl, a.zlo)) {
          const long long iz = ((long long)CpmlIdx::slot(gz, d.nz, Wl) * d.ny + j) * d.nx + i;
          const float ps = fmaf(__ldg(a.cz.b + gz), a.pqz[iz], __ldg(a.cz.a + gz) * dz);
          a.pqz[iz] = ps;
          dz += ps;
        }
      }
      float out = fmaf(kv, (dx + dy) + dz, pv);
      if (o == a.src_o) out += a.src_amp;
      a.p[o] = out;
      if (SNAP) a.snap[((long long)k * d.ny + j) * d.nx + i] = out;
    }
    __syncthreads();
    if (tid == 0 && it + AC_NS < np) {
      fence_proxy_async();
      mbar_expect_tx(&bar[s], TX_BYTES);
      tma_load_3d(sm + s * STAGE, &a.mqx, &bar[s], i0, j0 + G, k + AC_NS + G);
      tma_load_3d(sm + s * STAGE + TQX, &a.mqy, &bar[s], i0 + G, j0, k + AC_NS + G);
    }
    s0 = s1; s1 = s2; s2 = s3; s3 = s4; s4 = s5; s5 = s6; s6 = s7;
  }
}

}  // namespace seis
