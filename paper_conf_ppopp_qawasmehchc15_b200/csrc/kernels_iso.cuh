// kernels_iso.cuh — Eq 1: constant-density isotropic propagator.
//
//   u^{n+1} = [2u^n - (1 - eta dt) u^{n-1} + m Lambda u^n + s^n] / (1 + eta dt)
//   m = v^2 dt^2 / h^2 (per point, precomputed),  eta dt = edx[i] + edy[j] + edz[k]
//   Lambda u = 3 c0 u + sum_m c_m sum_axes (u_{+m} + u_{-m})         (O1, O3, O6)
//
// One thread per (x, y) column marching down a z-chunk (2.5D blocking).  Every
// operand of plane k arrives by TMA in one stage of an NS-deep mbarrier ring
// (the u^n tile with its x/y halo of 4, and the u^{n-1} and m tiles); the z
// neighbours come from a 9-deep register queue fed by a coalesced stream two
// planes ahead.  u^{n+1} overwrites u^{n-1} in place ("logically swapping
// t_n and t_{n+1} arrays").  HBM traffic per point: read u^n, u^{n-1}, m; write
// u^{n+1} = 16 B (+4 B snapshot, +12 B imaging).  Fused epilogues: source
// injection, snapshot store (O14), imaging I += S_j * u^n on
// the input level (O15).
#pragma once
#include "common.cuh"

namespace seis {

struct IsoArgs {
  CUtensorMap mun;               // u^n tile, box (32+8) x (BY+8) x 1
  CUtensorMap mup;               // u^{n-1}, box 32 x BY x 1
  CUtensorMap mm;                // m, box 32 x BY x 1
  const float* __restrict__ un;  // u^n (padded)
  float* __restrict__ up;        // out: u^{n+1} (in place of u^{n-1})
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

template <int BY>
struct IsoStage {
  static constexpr int W = TXW + 8;
  static constexpr int U = 0, UP = (BY + 8) * W, M = UP + TXW * BY, SIZE = M + TXW * BY;
  static constexpr size_t smem_bytes() { return (size_t)ISO_NS * SIZE * 4 + 128; }
};

template <int BY, bool SNAP, bool IMG>
__global__ void __launch_bounds__(TXW * BY) iso_step_kernel(const __grid_constant__ IsoArgs a) {
  using L = IsoStage<BY>;
  constexpr int W = L::W;
  constexpr uint32_t TX_BYTES = L::SIZE * 4;
  extern __shared__ __align__(128) float sm_raw[];
  float* sm = align128(sm_raw);
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
  auto issue = [&](int s, int k) {
    float* st = sm + s * L::SIZE;
    mbar_expect_tx(&bar[s], TX_BYTES);
    tma_load_3d(st + L::U, &a.mun, &bar[s], i0, j0, k + GZ);
    tma_load_3d(st + L::UP, &a.mup, &bar[s], i0 + G, j0 + G, k + GZ);
    tma_load_3d(st + L::M, &a.mm, &bar[s], i0 + G, j0 + G, k + GZ);
  };
  if (tid == 0) {
    for (int s = 0; s < ISO_NS; ++s) mbar_init(&bar[s], 1);
    mbar_fence_init();
  }
  __syncthreads();
  if (tid == 0)
    for (int s = 0; s < ISO_NS && s < np; ++s) issue(s, k0 + s);

  // z-queue u^n(k-4 .. k+4), fed two planes ahead
  float q0, q1, q2, q3, q4, q5, q6, q7, q8;
  q0 = __ldg(un + (long long)(k0 - 4 + GZ) * PS + oc);
  q1 = __ldg(un + (long long)(k0 - 3 + GZ) * PS + oc);
  q2 = __ldg(un + (long long)(k0 - 2 + GZ) * PS + oc);
  q3 = __ldg(un + (long long)(k0 - 1 + GZ) * PS + oc);
  q4 = __ldg(un + (long long)(k0 + GZ) * PS + oc);
  q5 = __ldg(un + (long long)(k0 + 1 + GZ) * PS + oc);
  q6 = __ldg(un + (long long)(k0 + 2 + GZ) * PS + oc);
  q7 = __ldg(un + (long long)(k0 + 3 + GZ) * PS + oc);
  float na = __ldg(un + (long long)(k0 + 4 + GZ) * PS + oc);
  float nb = np > 1 ? __ldg(un + (long long)(k0 + 5 + GZ) * PS + oc) : 0.f;
  const float exy = (a.edx && own) ? a.edx[i] + a.edy[j] : 0.0f;

  for (int it = 0; it < np; ++it) {
    const int k = k0 + it;
    const int s = it % ISO_NS;
    const long long o = (long long)(k + GZ) * PS + oc;
    q8 = na;
    na = nb;
    if (it + 2 < np) nb = __ldg(un + o + 6 * PS);
    mbar_wait(&bar[s], (it / ISO_NS) & 1);
    const float* st = sm + s * L::SIZE;
    const float* c = st + L::U + (ty + 4) * W + tx + 4;
    const float upv = st[L::UP + tid], mv = st[L::M + tid];
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
      issue(s, k + ISO_NS);
    }
    q0 = q1; q1 = q2; q2 = q3; q3 = q4; q4 = q5; q5 = q6; q6 = q7; q7 = q8;
  }
}

}  // namespace seis
