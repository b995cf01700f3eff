// kernels_iso.cuh — Eq 1: constant-density isotropic propagator.
//
//   u^{n+1} = [2u^n - (1 - eta dt) u^{n-1} + m Lambda u^n + s^n] / (1 + eta dt)
//   m = v^2 dt^2 / h^2 (per point, precomputed),  eta dt = edx[i] + edy[j] + edz[k]
//   Lambda u = 3 c0 u + sum_m c_m sum_axes (u_{+m} + u_{-m})         (O1, O3, O6)
//
// One thread per (x, y) column marching down a z-chunk (2.5D blocking).  The
// x/y neighbours of plane k come from a shared-memory tile (halo 4) brought in
// by TMA through an NS-stage mbarrier ring; the z neighbours from a 9-deep
// register queue fed by a coalesced stream prefetched one plane ahead, like
// u^{n-1} and m.  u^{n+1} overwrites u^{n-1} in place ("logically
// swapping t_n and t_{n+1} arrays").  HBM traffic per point: read u^n, u^{n-1},
// m; write u^{n+1} = 16 B (+4 B snapshot, +12 B imaging).  Fused epilogues:
// source injection, snapshot store (O14), imaging
// I += S_j * u^n on the input level (O15).
#pragma once
#include "common.cuh"

namespace seis {

struct IsoArgs {
  CUtensorMap mun;               // u^n, box (32+8) x (BY+8) x 1
  const float* __restrict__ un;  // u^n (padded)
  float* __restrict__ up;        // in: u^{n-1}; out: u^{n+1}
  const float* __restrict__ m;   // v^2 dt^2 / h^2 (padded)
  const float* __restrict__ edx; // eta*dt per axis (global index), nullptr = no layer
  const float* __restrict__ edy;
  const float* __restrict__ edz;
  Dims d;
  int zc;                        // z-chunk length
  long long src_o;               // padded index of the source node in this slab, -1 = none
  float src_amp;                 // scale * s[n]
  float* __restrict__ snap;      // compact [nzl][ny][nx] or nullptr
  const float* __restrict__ imgS;// compact snapshot S_j for imaging, or nullptr
  float* __restrict__ img;       // compact image (+=), or nullptr
};

constexpr int ISO_NS = 4;

template <int BY, bool SNAP, bool IMG>
__global__ void __launch_bounds__(TXW * BY) iso_step_kernel(const __grid_constant__ IsoArgs a) {
  constexpr int W = TXW + 8;
  constexpr int TILE = (BY + 8) * W;  // floats per stage (multiple of 32)
  constexpr uint32_t TX_BYTES = TILE * 4;
  __shared__ __align__(128) float sm[ISO_NS * TILE];
  __shared__ __align__(8) uint64_t bar[ISO_NS];
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
  const float* __restrict__ un = a.un;

  if (tid == 0) {
    for (int s = 0; s < ISO_NS; ++s) mbar_init(&bar[s], 1);
    mbar_fence_init();
  }
  __syncthreads();
  if (tid == 0) {
    for (int s = 0; s < ISO_NS && s < np; ++s) {
      mbar_expect_tx(&bar[s], TX_BYTES);
      tma_load_3d(sm + s * TILE, &a.mun, &bar[s], i0, j0, k0 + s + G);
    }
  }
  // z-queue u^n(k-4 .. k+4) and the one-plane-ahead streams
  float q0, q1, q2, q3, q4, q5, q6, q7, q8;
  q0 = __ldg(un + (long long)(k0 - 4 + G) * PS + oc);
  q1 = __ldg(un + (long long)(k0 - 3 + G) * PS + oc);
  q2 = __ldg(un + (long long)(k0 - 2 + G) * PS + oc);
  q3 = __ldg(un + (long long)(k0 - 1 + G) * PS + oc);
  q4 = __ldg(un + (long long)(k0 + G) * PS + oc);
  q5 = __ldg(un + (long long)(k0 + 1 + G) * PS + oc);
  q6 = __ldg(un + (long long)(k0 + 2 + G) * PS + oc);
  q7 = __ldg(un + (long long)(k0 + 3 + G) * PS + oc);
  float q8n = __ldg(un + (long long)(k0 + 4 + G) * PS + oc);
  float upn = 0.f, mn = 0.f;
  {
    const long long o = (long long)(k0 + G) * PS + oc;
    if (own && np > 0) {
      upn = a.up[o];
      mn = __ldg(a.m + o);
    }
  }
  const float exy = (a.edx && own) ? a.edx[i] + a.edy[j] : 0.0f;

  for (int it = 0; it < np; ++it) {
    const int k = k0 + it;
    const int s = it % ISO_NS;
    const long long o = (long long)(k + G) * PS + oc;
    q8 = q8n;
    const float upv = upn, mv = mn;
    if (it + 1 < np) {
      q8n = __ldg(un + o + 5 * PS);
      if (own) {
        upn = a.up[o + PS];
        mn = __ldg(a.m + o + PS);
      }
    }
    mbar_wait(&bar[s], (it / ISO_NS) & 1);
    const float* c = sm + s * TILE + (ty + 4) * W + tx + 4;
    float lap = (3.0f * SEIS_C0) * q4;
    lap = fmaf(SEIS_C1, (c[-1] + c[1]) + (c[-W] + c[W]) + (q3 + q5), lap);
    lap = fmaf(SEIS_C2, (c[-2] + c[2]) + (c[-2 * W] + c[2 * W]) + (q2 + q6), lap);
    lap = fmaf(SEIS_C3, (c[-3] + c[3]) + (c[-3 * W] + c[3 * W]) + (q1 + q7), lap);
    lap = fmaf(SEIS_C4, (c[-4] + c[4]) + (c[-4 * W] + c[4 * W]) + (q0 + q8), lap);
    if (own) {
      const float e = a.edx ? exy + a.edz[k + d.z0] : 0.0f;
      float out;
      if (e != 0.0f) {
        out = (2.0f * q4 - (1.0f - e) * upv + mv * lap) / (1.0f + e);
      } else {
        out = fmaf(mv, lap, 2.0f * q4 - upv);
      }
      if (o == a.src_o) out += a.src_amp;
      a.up[o] = out;
      if (SNAP || IMG) {
        const long long cix = ((long long)k * d.ny + j) * d.nx + i;
        if (SNAP) a.snap[cix] = out;
        if (IMG) a.img[cix] = fmaf(__ldg(a.imgS + cix), q4, a.img[cix]);
      }
    }
    __syncthreads();  // every thread is done with stage s
    if (tid == 0 && it + ISO_NS < np) {
      fence_proxy_async();
      mbar_expect_tx(&bar[s], TX_BYTES);
      tma_load_3d(sm + s * TILE, &a.mun, &bar[s], i0, j0, k + ISO_NS + G);
    }
    q0 = q1; q1 = q2; q2 = q3; q3 = q4; q4 = q5; q5 = q6; q6 = q7; q7 = q8;
  }
}

}  // namespace seis
