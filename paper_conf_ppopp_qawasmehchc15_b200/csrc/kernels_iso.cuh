// kernels_iso.cuh — Eq 1: constant-density isotropic propagator.
//
//   u^{n+1} = [2u^n - (1 - eta dt) u^{n-1} + m Lambda u^n + s^n] / (1 + eta dt)
//   m = v^2 dt^2 / h^2 (per point, precomputed),  eta dt = edx[i] + edy[j] + edz[k]
//   Lambda u = 3 c0 u + sum_m c_m sum_axes (u_{+m} + u_{-m})         (O1, O3, O6)
//
// One thread per (x, y) column marching down a z-chunk (2.5D blocking): the
// x/y neighbours of plane k come from a shared-memory tile (halo 4), the
// z neighbours from a 9-deep register queue.  u^{n+1} overwrites u^{n-1} in
// place ("logically swapping t_n and t_{n+1} arrays").  HBM traffic per
// point: read u^n, u^{n-1}, m; write u^{n+1} = 16 B (+4 B snapshot, +12 B imaging).
// Fused epilogues: source injection, snapshot store (O14),
// imaging I += S_j * u^n on the input level (O15).
#pragma once
#include "common.cuh"

namespace seis {

struct IsoArgs {
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

template <int BY, bool SNAP, bool IMG>
__global__ void __launch_bounds__(TXW * BY) iso_step_kernel(const IsoArgs a) {
  constexpr int W = TXW + 8;
  __shared__ float s[(BY + 8) * W];
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
  const float* __restrict__ un = a.un;

  float q0, q1, q2, q3, q4, q5, q6, q7, q8;  // u^n at k-4 .. k+4
  q0 = __ldg(un + (long long)(k0 - 4 + G) * PS + oc);
  q1 = __ldg(un + (long long)(k0 - 3 + G) * PS + oc);
  q2 = __ldg(un + (long long)(k0 - 2 + G) * PS + oc);
  q3 = __ldg(un + (long long)(k0 - 1 + G) * PS + oc);
  q4 = __ldg(un + (long long)(k0 + G) * PS + oc);
  q5 = __ldg(un + (long long)(k0 + 1 + G) * PS + oc);
  q6 = __ldg(un + (long long)(k0 + 2 + G) * PS + oc);
  q7 = __ldg(un + (long long)(k0 + 3 + G) * PS + oc);
  const float ex = (a.edx && own) ? a.edx[i] + a.edy[j] : 0.0f;

  for (int k = k0; k < k1; ++k) {
    const long long o = (long long)(k + G) * PS + oc;
    q8 = __ldg(un + o + 4 * PS);
    float upv = 0.0f, mv = 0.0f;
    if (own) {
      upv = a.up[o];
      mv = __ldg(a.m + o);
    }
    load_tile<BY, 4, 4>(s, un, (long long)(k + G) * PS + ot, d.PX);
    __syncthreads();
    const float* c = s + (ty + 4) * W + tx + 4;
    float lap = (3.0f * SEIS_C0) * q4;
    lap = fmaf(SEIS_C1, (c[-1] + c[1]) + (c[-W] + c[W]) + (q3 + q5), lap);
    lap = fmaf(SEIS_C2, (c[-2] + c[2]) + (c[-2 * W] + c[2 * W]) + (q2 + q6), lap);
    lap = fmaf(SEIS_C3, (c[-3] + c[3]) + (c[-3 * W] + c[3 * W]) + (q1 + q7), lap);
    lap = fmaf(SEIS_C4, (c[-4] + c[4]) + (c[-4 * W] + c[4 * W]) + (q0 + q8), lap);
    if (own) {
      const float e = a.edx ? ex + a.edz[k + d.z0] : 0.0f;
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
    __syncthreads();
    q0 = q1; q1 = q2; q2 = q3; q3 = q4; q4 = q5; q5 = q6; q6 = q7; q7 = q8;
  }
}

}  // namespace seis
