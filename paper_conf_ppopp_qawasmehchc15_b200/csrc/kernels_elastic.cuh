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
// psi stored times h (unscaled differences).  Free surface (O16): the top ghost
// planes hold the mirror images (filled by fs_mirror_kernel after every
// exchange), the surface row uses ezz = -lam/(lam+2mu)(exx+eyy), and szz = 0 on
// k = 0 after the source.
#pragma once
#include "common.cuh"
#include "kernels_acoustic.cuh"  // CpmlAxis

namespace seis {

enum { EVX, EVY, EVZ, ESXX, ESYY, ESZZ, ESXY, ESXZ, ESYZ };

__device__ __forceinline__ void cpml_x(float& dv, float* __restrict__ ps, const Dims& d, int W, int i,
                                       int j, int k, const float* __restrict__ ca,
                                       const float* __restrict__ cb) {
  const long long ix = ((long long)k * d.ny + j) * (2 * W) + CpmlIdx::slot(i, d.nx, W);
  const float v = fmaf(__ldg(cb + i), ps[ix], __ldg(ca + i) * dv);
  ps[ix] = v;
  dv += v;
}
__device__ __forceinline__ void cpml_y(float& dv, float* __restrict__ ps, const Dims& d, int W, int i,
                                       int j, int k, const float* __restrict__ ca,
                                       const float* __restrict__ cb) {
  const long long iy = ((long long)k * (2 * W) + CpmlIdx::slot(j, d.ny, W)) * d.nx + i;
  const float v = fmaf(__ldg(cb + j), ps[iy], __ldg(ca + j) * dv);
  ps[iy] = v;
  dv += v;
}
__device__ __forceinline__ void cpml_z(float& dv, float* __restrict__ ps, const Dims& d, int W, int i,
                                       int j, int gz, const float* __restrict__ ca,
                                       const float* __restrict__ cb) {
  const long long iz = ((long long)CpmlIdx::slot(gz, d.nz, W) * d.ny + j) * d.nx + i;
  const float v = fmaf(__ldg(cb + gz), ps[iz], __ldg(ca + gz) * dv);
  ps[iz] = v;
  dv += v;
}

// staggered differences on a shared-memory row/column (stride S), times h
template <int S>
__device__ __forceinline__ float dplus(const float* c) {  // at i+1/2 from integer field
  float r = SEIS_D1 * (c[S] - c[0]);
  r = fmaf(SEIS_D2, c[2 * S] - c[-S], r);
  r = fmaf(SEIS_D3, c[3 * S] - c[-2 * S], r);
  return fmaf(SEIS_D4, c[4 * S] - c[-3 * S], r);
}
template <int S>
__device__ __forceinline__ float dminus(const float* c) {  // at i from half field
  float r = SEIS_D1 * (c[0] - c[-S]);
  r = fmaf(SEIS_D2, c[S] - c[-2 * S], r);
  r = fmaf(SEIS_D3, c[2 * S] - c[-3 * S], r);
  return fmaf(SEIS_D4, c[3 * S] - c[-4 * S], r);
}
// z-queue versions: qp[0..7] = f(k-3 .. k+4) for D+, qm[0..7] = f(k-4 .. k+3) for D-
__device__ __forceinline__ float zplus(const float* q) {
  float r = SEIS_D1 * (q[4] - q[3]);
  r = fmaf(SEIS_D2, q[5] - q[2], r);
  r = fmaf(SEIS_D3, q[6] - q[1], r);
  return fmaf(SEIS_D4, q[7] - q[0], r);
}
__device__ __forceinline__ float zminus(const float* q) {
  float r = SEIS_D1 * (q[4] - q[3]);
  r = fmaf(SEIS_D2, q[5] - q[2], r);
  r = fmaf(SEIS_D3, q[6] - q[1], r);
  return fmaf(SEIS_D4, q[7] - q[0], r);
}

constexpr int EL_NS = 3;

struct ElVArgs {
  CUtensorMap msxx;  // box 40 x BY      (x halo)
  CUtensorMap msxy;  // box 40 x (BY+8)  (x and y halos)
  CUtensorMap msxz;  // box 40 x BY
  CUtensorMap msyy;  // box 32 x (BY+8)  (y halo)
  CUtensorMap msyz;  // box 32 x (BY+8)
  CUtensorMap mv[3]; // vx, vy, vz, box 32 x BY
  CUtensorMap mb[3]; // face buoyancies, box 32 x BY
  float* f[9];
  int W, zlo, fs;
  CpmlAxis cx, cy, cz;
  float* psi[9];   // psi 0..8
  Dims d;
  int zc;
};

template <int BY>
struct ElVStage {
  static constexpr int WX = TXW + 8, T = TXW * BY;
  static constexpr int XX = 0, XY = XX + BY * WX, XZ = XY + (BY + 8) * WX, YY = XZ + BY * WX,
                       YZ = YY + (BY + 8) * TXW, V = YZ + (BY + 8) * TXW, B = V + 3 * T, SIZE = B + 3 * T;
  static constexpr size_t smem_bytes() { return (size_t)EL_NS * SIZE * 4 + 128; }
};

template <int BY>
__global__ void __launch_bounds__(TXW * BY) el_v_kernel(const __grid_constant__ ElVArgs a) {
  using L = ElVStage<BY>;
  constexpr int WX = L::WX, T = L::T;
  constexpr uint32_t TX_BYTES = L::SIZE * 4;
  static_assert((L::XY % 32) == 0 && (L::XZ % 32) == 0 && (L::YY % 32) == 0 && (L::V % 32) == 0,
                "128-byte tiles");
  extern __shared__ __align__(128) float sm_raw[];
  float* sm = align128(sm_raw);
  __shared__ __align__(8) uint64_t bar[EL_NS];
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
  const int W = a.W;
  const bool lx = W > 0 && CpmlIdx::in(i, d.nx, W, true);
  const bool ly = W > 0 && CpmlIdx::in(j, d.ny, W, true);
  const float* __restrict__ sxz = a.f[ESXZ];
  const float* __restrict__ syz = a.f[ESYZ];
  const float* __restrict__ szz = a.f[ESZZ];
  auto issue = [&](int s, int k) {
    float* st = sm + s * L::SIZE;
    const int z = k + GZ;
    mbar_expect_tx(&bar[s], TX_BYTES);
    tma_load_3d(st + L::XX, &a.msxx, &bar[s], i0, j0 + G, z);
    tma_load_3d(st + L::XY, &a.msxy, &bar[s], i0, j0, z);
    tma_load_3d(st + L::XZ, &a.msxz, &bar[s], i0, j0 + G, z);
    tma_load_3d(st + L::YY, &a.msyy, &bar[s], i0 + G, j0, z);
    tma_load_3d(st + L::YZ, &a.msyz, &bar[s], i0 + G, j0, z);
#pragma unroll
    for (int c = 0; c < 3; ++c) {
      tma_load_3d(st + L::V + c * T, &a.mv[c], &bar[s], i0 + G, j0 + G, z);
      tma_load_3d(st + L::B + c * T, &a.mb[c], &bar[s], i0 + G, j0 + G, z);
    }
  };
  if (tid == 0) {
    for (int s = 0; s < EL_NS; ++s) mbar_init(&bar[s], 1);
    mbar_fence_init();
  }
  __syncthreads();
  if (tid == 0)
    for (int s = 0; s < EL_NS && s < np; ++s) issue(s, k0 + s);
  float qxz[8], qyz[8], qzz[8];  // sxz, syz at k-4..k+3 (D-); szz at k-3..k+4 (D+)
#pragma unroll
  for (int t = 0; t < 7; ++t) {
    qxz[t] = __ldg(sxz + (long long)(k0 - 4 + t + GZ) * PS + oc);
    qyz[t] = __ldg(syz + (long long)(k0 - 4 + t + GZ) * PS + oc);
    qzz[t] = __ldg(szz + (long long)(k0 - 3 + t + GZ) * PS + oc);
  }
  float axz = __ldg(sxz + (long long)(k0 + 3 + GZ) * PS + oc);
  float ayz = __ldg(syz + (long long)(k0 + 3 + GZ) * PS + oc);
  float azz = __ldg(szz + (long long)(k0 + 4 + GZ) * PS + oc);
  float bxz = 0.f, byz = 0.f, bzz = 0.f;
  if (np > 1) {
    bxz = __ldg(sxz + (long long)(k0 + 4 + GZ) * PS + oc);
    byz = __ldg(syz + (long long)(k0 + 4 + GZ) * PS + oc);
    bzz = __ldg(szz + (long long)(k0 + 5 + GZ) * PS + oc);
  }
  for (int it = 0; it < np; ++it) {
    const int k = k0 + it;
    const int s = it % EL_NS;
    const long long o = (long long)(k + GZ) * PS + oc;
    qxz[7] = axz; qyz[7] = ayz; qzz[7] = azz;
    axz = bxz; ayz = byz; azz = bzz;
    if (it + 2 < np) {
      bxz = __ldg(sxz + o + 5 * PS);
      byz = __ldg(syz + o + 5 * PS);
      bzz = __ldg(szz + o + 6 * PS);
    }
    mbar_wait(&bar[s], (it / EL_NS) & 1);
    if (own) {
      const float* st = sm + s * L::SIZE;
      const float* cxx = st + L::XX + ty * WX + tx + 4;
      const float* cxy = st + L::XY + (ty + 4) * WX + tx + 4;
      const float* cxz = st + L::XZ + ty * WX + tx + 4;
      const float* cyy = st + L::YY + (ty + 4) * TXW + tx;
      const float* cyz = st + L::YZ + (ty + 4) * TXW + tx;
      float d0 = dplus<1>(cxx), d1 = dminus<WX>(cxy), d2 = zminus(qxz);
      float d3 = dminus<1>(cxy), d4 = dplus<TXW>(cyy), d5 = zminus(qyz);
      float d6 = dminus<1>(cxz), d7 = dminus<TXW>(cyz), d8 = zplus(qzz);
      if (W > 0) {
        const int gz = k + d.z0;
        if (lx) {
          cpml_x(d0, a.psi[0], d, W, i, j, k, a.cx.ah, a.cx.bh);
          cpml_x(d3, a.psi[3], d, W, i, j, k, a.cx.a, a.cx.b);
          cpml_x(d6, a.psi[6], d, W, i, j, k, a.cx.a, a.cx.b);
        }
        if (ly) {
          cpml_y(d1, a.psi[1], d, W, i, j, k, a.cy.a, a.cy.b);
          cpml_y(d4, a.psi[4], d, W, i, j, k, a.cy.ah, a.cy.bh);
          cpml_y(d7, a.psi[7], d, W, i, j, k, a.cy.a, a.cy.b);
        }
        if (CpmlIdx::in(gz, d.nz, W, a.zlo)) {
          cpml_z(d2, a.psi[2], d, W, i, j, gz, a.cz.a, a.cz.b);
          cpml_z(d5, a.psi[5], d, W, i, j, gz, a.cz.a, a.cz.b);
          cpml_z(d8, a.psi[8], d, W, i, j, gz, a.cz.ah, a.cz.bh);
        }
      }
      const float* sv = st + L::V + tid;
      const float* sb = st + L::B + tid;
      a.f[EVX][o] = fmaf(sb[0], (d0 + d1) + d2, sv[0]);
      a.f[EVY][o] = fmaf(sb[T], (d3 + d4) + d5, sv[T]);
      a.f[EVZ][o] = fmaf(sb[2 * T], (d6 + d7) + d8, sv[2 * T]);
    }
    __syncthreads();
    if (tid == 0 && it + EL_NS < np) {
      fence_proxy_async();
      issue(s, k + EL_NS);
    }
#pragma unroll
    for (int t = 0; t < 7; ++t) {
      qxz[t] = qxz[t + 1];
      qyz[t] = qyz[t + 1];
      qzz[t] = qzz[t + 1];
    }
  }
}

struct ElSArgs {
  CUtensorMap mvt[3];  // vx, vy, vz tiles, box 40 x (BY+8)
  CUtensorMap ms[6];   // sxx, syy, szz, sxy, sxz, syz, box 32 x BY
  CUtensorMap mc[5];   // l2m, lam, mxy, mxz, myz, box 32 x BY
  float* f[9];
  int W, zlo, fs;
  CpmlAxis cx, cy, cz;
  float* psi[9];   // psi 9..17
  Dims d;
  int zc;
  long long src_o;
  float src_amp;   // dt (lam + 2/3 mu)_s / h^3 * s[n]
};

template <int BY>
struct ElSStage {
  static constexpr int WX = TXW + 8, T = TXW * BY, TV = (BY + 8) * WX;
  static constexpr int VT = 0, S = 3 * TV, C = S + 6 * T, SIZE = C + 5 * T;
  static constexpr size_t smem_bytes() { return (size_t)EL_NS * SIZE * 4 + 128; }
};

template <int BY, bool UNUSED>
__global__ void __launch_bounds__(TXW * BY) el_s_kernel(const __grid_constant__ ElSArgs a) {
  using L = ElSStage<BY>;
  constexpr int WX = L::WX, T = L::T, TV = L::TV;
  constexpr uint32_t TX_BYTES = L::SIZE * 4;
  extern __shared__ __align__(128) float sm_raw[];
  float* sm = align128(sm_raw);
  __shared__ __align__(8) uint64_t bar[EL_NS];
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
  const int W = a.W;
  const bool lx = W > 0 && CpmlIdx::in(i, d.nx, W, true);
  const bool ly = W > 0 && CpmlIdx::in(j, d.ny, W, true);
  const float* __restrict__ vx = a.f[EVX];
  const float* __restrict__ vy = a.f[EVY];
  const float* __restrict__ vz = a.f[EVZ];
  auto issue = [&](int s, int k) {
    float* st = sm + s * L::SIZE;
    const int z = k + GZ;
    mbar_expect_tx(&bar[s], TX_BYTES);
#pragma unroll
    for (int c = 0; c < 3; ++c) tma_load_3d(st + L::VT + c * TV, &a.mvt[c], &bar[s], i0, j0, z);
#pragma unroll
    for (int c = 0; c < 6; ++c) tma_load_3d(st + L::S + c * T, &a.ms[c], &bar[s], i0 + G, j0 + G, z);
#pragma unroll
    for (int c = 0; c < 5; ++c) tma_load_3d(st + L::C + c * T, &a.mc[c], &bar[s], i0 + G, j0 + G, z);
  };
  if (tid == 0) {
    for (int s = 0; s < EL_NS; ++s) mbar_init(&bar[s], 1);
    mbar_fence_init();
  }
  __syncthreads();
  if (tid == 0)
    for (int s = 0; s < EL_NS && s < np; ++s) issue(s, k0 + s);
  float qx[8], qy[8], qz[8];  // vx, vy at k-3..k+4 (D+); vz at k-4..k+3 (D-)
#pragma unroll
  for (int t = 0; t < 7; ++t) {
    qx[t] = __ldg(vx + (long long)(k0 - 3 + t + GZ) * PS + oc);
    qy[t] = __ldg(vy + (long long)(k0 - 3 + t + GZ) * PS + oc);
    qz[t] = __ldg(vz + (long long)(k0 - 4 + t + GZ) * PS + oc);
  }
  float ax = __ldg(vx + (long long)(k0 + 4 + GZ) * PS + oc);
  float ay = __ldg(vy + (long long)(k0 + 4 + GZ) * PS + oc);
  float az = __ldg(vz + (long long)(k0 + 3 + GZ) * PS + oc);
  float bx = 0.f, by = 0.f, bz = 0.f;
  if (np > 1) {
    bx = __ldg(vx + (long long)(k0 + 5 + GZ) * PS + oc);
    by = __ldg(vy + (long long)(k0 + 5 + GZ) * PS + oc);
    bz = __ldg(vz + (long long)(k0 + 4 + GZ) * PS + oc);
  }
  for (int it = 0; it < np; ++it) {
    const int k = k0 + it;
    const int s = it % EL_NS;
    const long long o = (long long)(k + GZ) * PS + oc;
    qx[7] = ax; qy[7] = ay; qz[7] = az;
    ax = bx; ay = by; az = bz;
    if (it + 2 < np) {
      bx = __ldg(vx + o + 6 * PS);
      by = __ldg(vy + o + 6 * PS);
      bz = __ldg(vz + o + 5 * PS);
    }
    mbar_wait(&bar[s], (it / EL_NS) & 1);
    if (own) {
      const int gz = k + d.z0;
      const float* st = sm + s * L::SIZE;
      const float* cvx = st + L::VT + (ty + 4) * WX + tx + 4;
      const float* cvy = cvx + TV;
      const float* cvz = cvx + 2 * TV;
      float exx = dminus<1>(cvx), eyy = dminus<WX>(cvy), ezz = zminus(qz);
      float dyvx = dplus<WX>(cvx), dxvy = dplus<1>(cvy);
      float dzvx = zplus(qx), dxvz = dplus<1>(cvz);
      float dzvy = zplus(qy), dyvz = dplus<WX>(cvz);
      if (W > 0) {
        if (lx) {
          cpml_x(exx, a.psi[0], d, W, i, j, k, a.cx.a, a.cx.b);
          cpml_x(dxvy, a.psi[4], d, W, i, j, k, a.cx.ah, a.cx.bh);
          cpml_x(dxvz, a.psi[6], d, W, i, j, k, a.cx.ah, a.cx.bh);
        }
        if (ly) {
          cpml_y(eyy, a.psi[1], d, W, i, j, k, a.cy.a, a.cy.b);
          cpml_y(dyvx, a.psi[3], d, W, i, j, k, a.cy.ah, a.cy.bh);
          cpml_y(dyvz, a.psi[8], d, W, i, j, k, a.cy.ah, a.cy.bh);
        }
        if (CpmlIdx::in(gz, d.nz, W, a.zlo)) {
          cpml_z(ezz, a.psi[2], d, W, i, j, gz, a.cz.a, a.cz.b);
          cpml_z(dzvx, a.psi[5], d, W, i, j, gz, a.cz.ah, a.cz.bh);
          cpml_z(dzvy, a.psi[7], d, W, i, j, gz, a.cz.ah, a.cz.bh);
        }
      }
      const float* ss = st + L::S + tid;
      const float* sc = st + L::C + tid;
      const float l2m = sc[0], lam = sc[T];
      const bool surf = a.fs && gz == 0;
      if (surf) ezz = -(lam / l2m) * (exx + eyy);  // O16 surface row
      float sxx = ss[0] + fmaf(l2m, exx, lam * (eyy + ezz));
      float syy = ss[T] + fmaf(l2m, eyy, lam * (exx + ezz));
      float szz = ss[2 * T] + fmaf(l2m, ezz, lam * (exx + eyy));
      if (o == a.src_o) {
        sxx -= a.src_amp;
        syy -= a.src_amp;
        szz -= a.src_amp;
      }
      if (surf) szz = 0.0f;
      a.f[ESXX][o] = sxx;
      a.f[ESYY][o] = syy;
      a.f[ESZZ][o] = szz;
      a.f[ESXY][o] = fmaf(sc[2 * T], dyvx + dxvy, ss[3 * T]);
      a.f[ESXZ][o] = fmaf(sc[3 * T], dzvx + dxvz, ss[4 * T]);
      a.f[ESYZ][o] = fmaf(sc[4 * T], dzvy + dyvz, ss[5 * T]);
    }
    __syncthreads();
    if (tid == 0 && it + EL_NS < np) {
      fence_proxy_async();
      issue(s, k + EL_NS);
    }
#pragma unroll
    for (int t = 0; t < 7; ++t) {
      qx[t] = qx[t + 1];
      qy[t] = qy[t + 1];
      qz[t] = qz[t + 1];
    }
  }
}

// Free-surface ghost planes above k = 0 (O16): for field f with parity `odd`
// (1: antisymmetric, 0: symmetric) and staggering `half` (1: z-half node),
//   integer z: ghost(-m) = +-f(m), m = 1..4;   half z: ghost(-1-m) = +-f(m), m = 0..3.
__global__ void fs_mirror_kernel(float* __restrict__ f, Dims d, int odd, int half) {
  const int i = blockIdx.x * blockDim.x + threadIdx.x;
  const int j = blockIdx.y;
  if (i >= d.nx) return;
  const float sgn = odd ? -1.0f : 1.0f;
#pragma unroll
  for (int m = 0; m < 4; ++m) {
    const int src = half ? m : m + 1;
    const int dst = half ? -1 - m : -(m + 1);
    f[d.at(i, j, dst)] = sgn * f[d.at(i, j, src)];
  }
}

}  // namespace seis
