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

struct ElVArgs {
  float* f[9];
  const float* __restrict__ bx;
  const float* __restrict__ by;
  const float* __restrict__ bz;
  int W, zlo, fs;
  CpmlAxis cx, cy, cz;
  float* psi[9];   // psi 0..8
  Dims d;
  int zc;
};

template <int BY>
__global__ void __launch_bounds__(TXW * BY) el_v_kernel(const ElVArgs a) {
  constexpr int WX = TXW + 8;
  __shared__ float t_sxx[BY * WX];          // x halo
  __shared__ float t_sxy[(BY + 8) * WX];    // x and y halos
  __shared__ float t_sxz[BY * WX];          // x halo
  __shared__ float t_syy[(BY + 8) * TXW];   // y halo
  __shared__ float t_syz[(BY + 8) * TXW];   // y halo
  const Dims& d = a.d;
  const int tx = threadIdx.x, ty = threadIdx.y;
  const int i0 = blockIdx.x * TXW, j0 = blockIdx.y * BY;
  const int i = i0 + tx, j = j0 + ty;
  const int k0 = blockIdx.z * a.zc;
  const int k1 = min(k0 + a.zc, d.nzl);
  const bool own = (i < d.nx) && (j < d.ny);
  const long long PS = d.PS;
  const long long oc = (long long)(j + G) * d.PX + (i + G);
  const long long ot = (long long)(j0 + G) * d.PX + (i0 + G);
  const int W = a.W;
  const bool lx = W > 0 && CpmlIdx::in(i, d.nx, W, true);
  const bool ly = W > 0 && CpmlIdx::in(j, d.ny, W, true);
  const float* __restrict__ sxz = a.f[ESXZ];
  const float* __restrict__ syz = a.f[ESYZ];
  const float* __restrict__ szz = a.f[ESZZ];
  float qxz[8], qyz[8], qzz[8];  // sxz, syz at k-4..k+3 (D-); szz at k-3..k+4 (D+)
#pragma unroll
  for (int t = 0; t < 7; ++t) {
    qxz[t] = __ldg(sxz + (long long)(k0 - 4 + t + G) * PS + oc);
    qyz[t] = __ldg(syz + (long long)(k0 - 4 + t + G) * PS + oc);
    qzz[t] = __ldg(szz + (long long)(k0 - 3 + t + G) * PS + oc);
  }
  for (int k = k0; k < k1; ++k) {
    const long long o = (long long)(k + G) * PS + oc;
    qxz[7] = __ldg(sxz + o + 3 * PS);
    qyz[7] = __ldg(syz + o + 3 * PS);
    qzz[7] = __ldg(szz + o + 4 * PS);
    const long long op = (long long)(k + G) * PS + ot;
    load_tile<BY, 4, 0>(t_sxx, a.f[ESXX], op, d.PX);
    load_tile<BY, 4, 4>(t_sxy, a.f[ESXY], op, d.PX);
    load_tile<BY, 4, 0>(t_sxz, a.f[ESXZ], op, d.PX);
    load_tile<BY, 0, 4>(t_syy, a.f[ESYY], op, d.PX);
    load_tile<BY, 0, 4>(t_syz, a.f[ESYZ], op, d.PX);
    __syncthreads();
    if (own) {
      const float* cxx = t_sxx + ty * WX + tx + 4;
      const float* cxy = t_sxy + (ty + 4) * WX + tx + 4;
      const float* cxz = t_sxz + ty * WX + tx + 4;
      const float* cyy = t_syy + (ty + 4) * TXW + tx;
      const float* cyz = t_syz + (ty + 4) * TXW + tx;
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
      a.f[EVX][o] = fmaf(__ldg(a.bx + o), (d0 + d1) + d2, a.f[EVX][o]);
      a.f[EVY][o] = fmaf(__ldg(a.by + o), (d3 + d4) + d5, a.f[EVY][o]);
      a.f[EVZ][o] = fmaf(__ldg(a.bz + o), (d6 + d7) + d8, a.f[EVZ][o]);
    }
    __syncthreads();
#pragma unroll
    for (int t = 0; t < 7; ++t) {
      qxz[t] = qxz[t + 1];
      qyz[t] = qyz[t + 1];
      qzz[t] = qzz[t + 1];
    }
  }
}

struct ElSArgs {
  float* f[9];
  const float* __restrict__ l2m;  // dt (lam + 2 mu) / h
  const float* __restrict__ lam;  // dt lam / h
  const float* __restrict__ mxy;  // dt mu_xy / h (edge, harmonic mean)
  const float* __restrict__ mxz;
  const float* __restrict__ myz;
  int W, zlo, fs;
  CpmlAxis cx, cy, cz;
  float* psi[9];   // psi 9..17
  Dims d;
  int zc;
  long long src_o;
  float src_amp;   // dt (lam + 2/3 mu)_s / h^3 * s[n]
};

template <int BY, bool UNUSED>
__global__ void __launch_bounds__(TXW * BY) el_s_kernel(const ElSArgs a) {
  constexpr int WX = TXW + 8;
  __shared__ float t_vx[(BY + 8) * WX];
  __shared__ float t_vy[(BY + 8) * WX];
  __shared__ float t_vz[(BY + 8) * WX];
  const Dims& d = a.d;
  const int tx = threadIdx.x, ty = threadIdx.y;
  const int i0 = blockIdx.x * TXW, j0 = blockIdx.y * BY;
  const int i = i0 + tx, j = j0 + ty;
  const int k0 = blockIdx.z * a.zc;
  const int k1 = min(k0 + a.zc, d.nzl);
  const bool own = (i < d.nx) && (j < d.ny);
  const long long PS = d.PS;
  const long long oc = (long long)(j + G) * d.PX + (i + G);
  const long long ot = (long long)(j0 + G) * d.PX + (i0 + G);
  const int W = a.W;
  const bool lx = W > 0 && CpmlIdx::in(i, d.nx, W, true);
  const bool ly = W > 0 && CpmlIdx::in(j, d.ny, W, true);
  const float* __restrict__ vx = a.f[EVX];
  const float* __restrict__ vy = a.f[EVY];
  const float* __restrict__ vz = a.f[EVZ];
  float qx[8], qy[8], qz[8];  // vx, vy at k-3..k+4 (D+); vz at k-4..k+3 (D-)
#pragma unroll
  for (int t = 0; t < 7; ++t) {
    qx[t] = __ldg(vx + (long long)(k0 - 3 + t + G) * PS + oc);
    qy[t] = __ldg(vy + (long long)(k0 - 3 + t + G) * PS + oc);
    qz[t] = __ldg(vz + (long long)(k0 - 4 + t + G) * PS + oc);
  }
  for (int k = k0; k < k1; ++k) {
    const long long o = (long long)(k + G) * PS + oc;
    qx[7] = __ldg(vx + o + 4 * PS);
    qy[7] = __ldg(vy + o + 4 * PS);
    qz[7] = __ldg(vz + o + 3 * PS);
    const long long op = (long long)(k + G) * PS + ot;
    load_tile<BY, 4, 4>(t_vx, vx, op, d.PX);
    load_tile<BY, 4, 4>(t_vy, vy, op, d.PX);
    load_tile<BY, 4, 4>(t_vz, vz, op, d.PX);
    __syncthreads();
    if (own) {
      const int gz = k + d.z0;
      const float* cvx = t_vx + (ty + 4) * WX + tx + 4;
      const float* cvy = t_vy + (ty + 4) * WX + tx + 4;
      const float* cvz = t_vz + (ty + 4) * WX + tx + 4;
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
      const float l2m = __ldg(a.l2m + o), lam = __ldg(a.lam + o);
      const bool surf = a.fs && gz == 0;
      if (surf) ezz = -(lam / l2m) * (exx + eyy);  // O16 surface row
      float sxx = a.f[ESXX][o], syy = a.f[ESYY][o], szz = a.f[ESZZ][o];
      sxx += fmaf(l2m, exx, lam * (eyy + ezz));
      syy += fmaf(l2m, eyy, lam * (exx + ezz));
      szz += fmaf(l2m, ezz, lam * (exx + eyy));
      if (o == a.src_o) {
        sxx -= a.src_amp;
        syy -= a.src_amp;
        szz -= a.src_amp;
      }
      if (surf) szz = 0.0f;
      a.f[ESXX][o] = sxx;
      a.f[ESYY][o] = syy;
      a.f[ESZZ][o] = szz;
      a.f[ESXY][o] = fmaf(__ldg(a.mxy + o), dyvx + dxvy, a.f[ESXY][o]);
      a.f[ESXZ][o] = fmaf(__ldg(a.mxz + o), dzvx + dxvz, a.f[ESXZ][o]);
      a.f[ESYZ][o] = fmaf(__ldg(a.myz + o), dzvy + dyvz, a.f[ESYZ][o]);
    }
    __syncthreads();
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
