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
  CUtensorMap mp;                 // p tile, box (32+8) x (BY+8) x 1
  CUtensorMap mqx, mqy, mqz;      // q, box 32 x BY x 1
  CUtensorMap mbx, mby, mbz;      // face buoyancy, box 32 x BY x 1
  const float* __restrict__ p;
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
  const float* __restrict__ imgS; // imaging: img += S * p (input level), or nullptr
  float* __restrict__ img;
};

template <int BY>
struct AcVStage {
  static constexpr int W = TXW + 8, T = TXW * BY;
  static constexpr int P = 0, QX = (BY + 8) * W, QY = QX + T, QZ = QY + T, BX = QZ + T, BYo = BX + T,
                       BZ = BYo + T, SIZE = BZ + T;
  static constexpr size_t smem_bytes() { return (size_t)AC_NS * SIZE * 4 + 128; }
};

template <int BY, bool IMG>
__global__ void __launch_bounds__(TXW * BY) ac_v_kernel(const __grid_constant__ AcVArgs a) {
  using L = AcVStage<BY>;
  constexpr int W = L::W;
  constexpr uint32_t TX_BYTES = L::SIZE * 4;
  extern __shared__ __align__(128) float sm_raw[];
  float* sm = align128(sm_raw);
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
  auto issue = [&](int s, int k) {
    float* st = sm + s * L::SIZE;
    const int z = k + G, x = i0 + G, y = j0 + G;
    mbar_expect_tx(&bar[s], TX_BYTES);
    tma_load_3d(st + L::P, &a.mp, &bar[s], i0, j0, z);
    tma_load_3d(st + L::QX, &a.mqx, &bar[s], x, y, z);
    tma_load_3d(st + L::QY, &a.mqy, &bar[s], x, y, z);
    tma_load_3d(st + L::QZ, &a.mqz, &bar[s], x, y, z);
    tma_load_3d(st + L::BX, &a.mbx, &bar[s], x, y, z);
    tma_load_3d(st + L::BYo, &a.mby, &bar[s], x, y, z);
    tma_load_3d(st + L::BZ, &a.mbz, &bar[s], x, y, z);
  };
  if (tid == 0) {
    for (int s = 0; s < AC_NS; ++s) mbar_init(&bar[s], 1);
    mbar_fence_init();
  }
  __syncthreads();
  if (tid == 0)
    for (int s = 0; s < AC_NS && s < np; ++s) issue(s, k0 + s);
  float r0, r1, r2, r3, r4, r5, r6, r7;  // p at k-3 .. k+4, fed two planes ahead
  r0 = __ldg(p + (long long)(k0 - 3 + G) * PS + oc);
  r1 = __ldg(p + (long long)(k0 - 2 + G) * PS + oc);
  r2 = __ldg(p + (long long)(k0 - 1 + G) * PS + oc);
  r3 = __ldg(p + (long long)(k0 + G) * PS + oc);
  r4 = __ldg(p + (long long)(k0 + 1 + G) * PS + oc);
  r5 = __ldg(p + (long long)(k0 + 2 + G) * PS + oc);
  r6 = __ldg(p + (long long)(k0 + 3 + G) * PS + oc);
  float na = __ldg(p + (long long)(k0 + 4 + G) * PS + oc);
  float nb = np > 1 ? __ldg(p + (long long)(k0 + 5 + G) * PS + oc) : 0.f;

  for (int it = 0; it < np; ++it) {
    const int k = k0 + it;
    const int s = it % AC_NS;
    const long long o = (long long)(k + G) * PS + oc;
    r7 = na;
    na = nb;
    if (it + 2 < np) nb = __ldg(p + o + 6 * PS);
    mbar_wait(&bar[s], (it / AC_NS) & 1);
    const float* st = sm + s * L::SIZE;
    const float* c = st + L::P + (ty + 4) * W + tx + 4;
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
      a.qx[o] = fmaf(st[L::BX + tid], dx, st[L::QX + tid]);
      a.qy[o] = fmaf(st[L::BYo + tid], dy, st[L::QY + tid]);
      a.qz[o] = fmaf(st[L::BZ + tid], dz, st[L::QZ + tid]);
      if (IMG) {
        const long long cix = ((long long)k * d.ny + j) * d.nx + i;
        a.img[cix] = fmaf(__ldg(a.imgS + cix), r3, a.img[cix]);
      }
    }
    __syncthreads();
    if (tid == 0 && it + AC_NS < np) {
      fence_proxy_async();
      issue(s, k + AC_NS);
    }
    r0 = r1; r1 = r2; r2 = r3; r3 = r4; r4 = r5; r5 = r6; r6 = r7;
  }
}

struct AcPArgs {
  CUtensorMap mqx;                // q_x, box (32+8) x BY x 1
  CUtensorMap mqy;                // q_y, box 32 x (BY+8) x 1
  CUtensorMap mpp;                // p, box 32 x BY x 1
  CUtensorMap mk;                 // dt K / h, box 32 x BY x 1
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
  long long src_o;                // padded index of the source in this slab, -1 = none
  float src_amp;                  // dt K_s / h^3 * s[n]
  float* __restrict__ snap;       // compact snapshot target, or nullptr
};

template <int BY>
struct AcPStage {
  static constexpr int WX = TXW + 8, T = TXW * BY;
  static constexpr int QX = 0, QY = BY * WX, P = QY + (BY + 8) * TXW, K = P + T, SIZE = K + T;
  static constexpr size_t smem_bytes() { return (size_t)AC_NS * SIZE * 4 + 128; }
};

template <int BY, bool SNAP>
__global__ void __launch_bounds__(TXW * BY) ac_p_kernel(const __grid_constant__ AcPArgs a) {
  using L = AcPStage<BY>;
  constexpr int WX = L::WX;
  constexpr uint32_t TX_BYTES = L::SIZE * 4;
  extern __shared__ __align__(128) float sm_raw[];
  float* sm = align128(sm_raw);
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
  auto issue = [&](int s, int k) {
    float* st = sm + s * L::SIZE;
    const int z = k + G;
    mbar_expect_tx(&bar[s], TX_BYTES);
    tma_load_3d(st + L::QX, &a.mqx, &bar[s], i0, j0 + G, z);
    tma_load_3d(st + L::QY, &a.mqy, &bar[s], i0 + G, j0, z);
    tma_load_3d(st + L::P, &a.mpp, &bar[s], i0 + G, j0 + G, z);
    tma_load_3d(st + L::K, &a.mk, &bar[s], i0 + G, j0 + G, z);
  };
  if (tid == 0) {
    for (int s = 0; s < AC_NS; ++s) mbar_init(&bar[s], 1);
    mbar_fence_init();
  }
  __syncthreads();
  if (tid == 0)
    for (int s = 0; s < AC_NS && s < np; ++s) issue(s, k0 + s);
  float s0, s1, s2, s3, s4, s5, s6, s7;  // q_z at k-4 .. k+3, fed two planes ahead
  s0 = __ldg(qz + (long long)(k0 - 4 + G) * PS + oc);
  s1 = __ldg(qz + (long long)(k0 - 3 + G) * PS + oc);
  s2 = __ldg(qz + (long long)(k0 - 2 + G) * PS + oc);
  s3 = __ldg(qz + (long long)(k0 - 1 + G) * PS + oc);
  s4 = __ldg(qz + (long long)(k0 + G) * PS + oc);
  s5 = __ldg(qz + (long long)(k0 + 1 + G) * PS + oc);
  s6 = __ldg(qz + (long long)(k0 + 2 + G) * PS + oc);
  float na = __ldg(qz + (long long)(k0 + 3 + G) * PS + oc);
  float nb = np > 1 ? __ldg(qz + (long long)(k0 + 4 + G) * PS + oc) : 0.f;

  for (int it = 0; it < np; ++it) {
    const int k = k0 + it;
    const int s = it % AC_NS;
    const long long o = (long long)(k + G) * PS + oc;
    s7 = na;
    na = nb;
    if (it + 2 < np) nb = __ldg(qz + o + 5 * PS);
    mbar_wait(&bar[s], (it / AC_NS) & 1);
    const float* st = sm + s * L::SIZE;
    const float* cx = st + L::QX + ty * WX + tx + 4;
    const float* cy = st + L::QY + (ty + 4) * TXW + tx;
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
      float out = fmaf(st[L::K + tid], (dx + dy) + dz, st[L::P + tid]);
      if (o == a.src_o) out += a.src_amp;
      a.p[o] = out;
      if (SNAP) a.snap[((long long)k * d.ny + j) * d.nx + i] = out;
    }
    __syncthreads();
    if (tid == 0 && it + AC_NS < np) {
      fence_proxy_async();
      issue(s, k + AC_NS);
    }
    s0 = s1; s1 = s2; s2 = s3; s3 = s4; s4 = s5; s5 = s6; s6 = s7;
  }
}

}  // namespace seis
