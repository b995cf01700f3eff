// kernels_iso.cuh — Eq 1: constant-density isotropic propagator.
//
//   u^{n+1} = [2u^n - (1 - eta dt) u^{n-1} + m Lambda u^n + s^n] / (1 + eta dt)
//   m = v^2 dt^2 / h^2 (per point, precomputed),  eta dt = edx[i] + edy[j] + edz[k]
//   Lambda u = 3 c0 u + sum_m c_m sum_axes (u_{+m} + u_{-m})         (O1, O3, O6)
//
// 2.5D z-march: a block owns a 64 x BY (x, y) tile and walks a z-chunk; each
// thread owns 4 consecutive x points (one float4).  Every operand of plane k
// arrives by TMA in one stage of an NS-deep mbarrier ring: the u^n tile with
// its x/y halo of 4 (x-neighbours from three 16-byte shared loads per row,
// y-neighbours from eight), the u^{n-1} and m tiles, and the interior tile of
// u^n at plane k+4 that feeds the 9-deep float4 register queue of z neighbours
// (no global load in the z-march except the queue warm-up).  u^{n+1} overwrites u^{n-1} in place ("logically swapping t_n and
// t_{n+1} arrays").  HBM traffic per point: read u^n, u^{n-1}, m; write u^{n+1}
// = 16 B (+4 B snapshot, +12 B imaging).  Fused epilogues: source injection
// (P:191), snapshot store (O14), imaging I += S_j * u^n on the input
// level (O15).
#pragma once
#include "common.cuh"

#ifndef SEIS_ISO_RCP
#define SEIS_ISO_RCP 1  // profiles/r01_sweep_zu.jsonl: iso_step 0.429 -> 0.370 ms at 512^3
#endif

namespace seis {

// Eq 1 / O3 per point, shared by the z-march kernel and the persistent small-grid kernel so
// both contract and round identically (bitwise equal results):
// 25-point Laplacian x h^2 of O1 from the ring pair sums xs[m], ys[m], zs[m] (m = 1..4) ...
__device__ __forceinline__ float iso_lap(float u, const float* xs, const float* ys, const float* zs) {
  float l = (3.0f * SEIS_C0) * u;
  l = fmaf(SEIS_C1, (xs[0] + ys[0]) + zs[0], l);
  l = fmaf(SEIS_C2, (xs[1] + ys[1]) + zs[1], l);
  l = fmaf(SEIS_C3, (xs[2] + ys[2]) + zs[2], l);
  return fmaf(SEIS_C4, (xs[3] + ys[3]) + zs[3], l);
}
// ... and the leapfrog update with the damped-wave layer (eta = eta dt; 0 outside)
__device__ __forceinline__ float iso_update(float u, float up, float m, float lap, float eta) {
  if (eta == 0.0f) return fmaf(m, lap, 2.0f * u - up);
#if SEIS_ISO_RCP
  // MUFU reciprocal + one Newton step (~0.5 ulp) instead of the IEEE division
  const float den = 1.0f + eta;
  float inv = rcp_fast(den);
  inv = fmaf(inv, fmaf(-den, inv, 1.0f), inv);
  return (2.0f * u - (1.0f - eta) * up + m * lap) * inv;
#else
  return (2.0f * u - (1.0f - eta) * up + m * lap) / (1.0f + eta);
#endif
}

struct IsoArgs {
  CUtensorMap mun;               // u^n tile, box (64+8) x (BY+8) x 1
  CUtensorMap mup;               // u^{n-1}, box 64 x BY x 1
  CUtensorMap mm;                // m, box 64 x BY x 1
  CUtensorMap muq;               // u^n interior tile (z-queue feed, plane k+4), box 64 x BY x 1
  const float* __restrict__ un;  // u^n (padded)
  float* __restrict__ up;        // out: u^{n+1} (in place of u^{n-1})
  const float* __restrict__ edx; // eta*dt per axis (global index, padded to PX), nullptr = no layer
  const float* __restrict__ edy;
  const float* __restrict__ edz;
  Dims d;
  int zc;                        // z-chunk length
  int ch0, chs;                  // z-chunk of blockIdx.z = ch0 + blockIdx.z * chs (boundary / interior split)
  // Region split of the split-field PML step (O6b): 0 = every block; 1 = only blocks whose tile
  // and z-chunk hold no layer point (the plain kernel, high occupancy); 2 = only the other
  // blocks (the SPML kernel).  nbr = layer width (points) for the test.
  int region, nbr;
  long long src_o;               // padded index of the source node in this slab, -1 = none
  SrcAmp src;                    // scale * s[n]
  float* __restrict__ snap;      // compact [nzl][ny][nx] or nullptr
  const float* __restrict__ imgS;// compact snapshot S_j for imaging, or nullptr
  SnapRef imgR;                  // the same (fp32 or 24-bit), what the IMG kernels read
  float* __restrict__ img;       // compact image (+=), or nullptr
  Ghost gh;                      // direct ghost stores of u^{n+1} (f4)
  // split-field PML (O6b, SPML kernels): components u^(x), u^(y), u^(z) of the layer points,
  // compact storage sp[(lvl * 3 + d) * spn + idx], lvl = time level (u^n: lvl, u^{n-1} and
  // the new u^{n+1}: 1 - lvl), idx = x-slab [nzl][ny][2nb] for points in the x layer, else
  // y-slab [nzl][2nb][nx] (offset nxs), else z-slab [2nb][ny][nx] (global z slot, offset nxs + nys)
  float* __restrict__ sp;
  long long spn;
  int nbl, nxs, nys, lvl;
  // per-axis update coefficients [3][spnp[axis]] (A, B, C of the component update, host-rounded)
  const float* __restrict__ spco[3];
  int spnp[3];
};

// O6b storage index of a layer point (ex / ey: eta_x dt, eta_y dt at the point)
__device__ __forceinline__ int spml_idx(const Dims& d, int nb, int nxs, int nys, float ex, float ey, int x, int j,
                                        int k) {
  if (ex != 0.0f) return (k * d.ny + j) * (2 * nb) + (x < nb ? x : x - (d.nx - 2 * nb));
  if (ey != 0.0f) return nxs + (k * (2 * nb) + (j < nb ? j : j - (d.ny - 2 * nb))) * d.nx + x;
  const int gz = k + d.z0;
  return nxs + nys + ((gz < nb ? gz : gz - (d.nz - 2 * nb)) * d.ny + j) * d.nx + x;
}

#ifndef SEIS_SPML_MINB
#define SEIS_SPML_MINB 3  // O6b kernels: >= 3 resident blocks (<= 170 registers; 0.762 vs 0.974 ms)
#endif
#ifndef SEIS_ISO_NS
#define SEIS_ISO_NS 3
#endif
// O6b layer components by cp.async two planes ahead into per-thread shared slots, instead of
// register loads issued one plane ahead (whose latency is the kernel's top stall): measured
// and rejected, off -- 0.853 vs 0.739 ms at 512^3 (profiles/r02_iso_pml_variants.txt)
#ifndef SEIS_SPML_PF
#define SEIS_SPML_PF 0
#endif
// (O6b) L2 prefetch of the layer components SEIS_SPML_PSIPF planes ahead (0 = off): one lane
// per 8 (a 128-byte line of a y / z slab row), the group's first point
#ifndef SEIS_SPML_PSIPF
#define SEIS_SPML_PSIPF 1  // 0.715 -> 0.697 ms at 512^3 (70 % of HBM; 2: 0.697, 3: 0.699), profiles/r02_spml_psipf.log
#endif
constexpr int ISO_NS = SEIS_ISO_NS;

template <int BY>
struct IsoStage {
  static constexpr int W = TXV + 8;
  static constexpr int U = 0, UP = (BY + 8) * W, M = UP + TXV * BY, UQ = M + TXV * BY, SIZE = UQ + TXV * BY;
  static constexpr size_t smem_bytes() { return (size_t)ISO_NS * SIZE * 4 + 128; }
  // (SPML, SEIS_SPML_PF) + per-thread slots: 3 planes x 6 component arrays x 4 points
  static constexpr int CSLOT = 3 * 6 * NTX * BY * 4;
  static constexpr size_t smem_bytes_spml() { return smem_bytes() + (SEIS_SPML_PF ? (size_t)CSLOT * 4 : 0); }
};

// Launch bounds: an explicit minimum of 1 block lets ptxas give the plain kernel 96 registers
// instead of 80 -- 0.370 -> 0.345 ms at 512^3 (profiles/r01_sweep_zu.jsonl).
// GH: this slab has a neighbour slab / rank whose ghost planes it stores (f4); the single-slab
// instantiation leaves the check out (-2.7 % iso_step time, profiles/r01_sweep_zu.jsonl)
template <int BY, bool SNAP, bool IMG, bool SPML = false, bool GH = true>
__global__ void __launch_bounds__(NTX * BY, SPML ? SEIS_SPML_MINB : 1) iso_step_kernel(const __grid_constant__ IsoArgs a) {
  using L = IsoStage<BY>;
  constexpr int W = L::W;
  constexpr uint32_t TX_BYTES = L::SIZE * 4;
  extern __shared__ __align__(128) float sm_raw[];
  float* sm = align128(sm_raw);
  __shared__ __align__(8) uint64_t bar[ISO_NS];
  __shared__ uint32_t cnt[ISO_NS];
  const Dims& d = a.d;
  const int tx = threadIdx.x, ty = threadIdx.y, tid = ty * NTX + tx;
  const int i0 = blockIdx.x * TXV, j0 = blockIdx.y * BY;
  const int x0 = i0 + 4 * tx, j = j0 + ty;
  const int k0 = (a.ch0 + (int)blockIdx.z * a.chs) * a.zc;
  const int k1 = min(k0 + a.zc, d.nzl);
  const int np = k1 - k0;
  if (a.region) {  // block-uniform: is this block's (tile, chunk) free of layer points?
    const int nb = a.nbr;
    const bool inner = i0 >= nb && min(i0 + TXV, d.nx) - 1 <= d.nx - 1 - nb && j0 >= nb &&
                       min(j0 + BY, d.ny) - 1 <= d.ny - 1 - nb && k0 + d.z0 >= nb && k1 - 1 + d.z0 <= d.nz - 1 - nb;
    if (inner != (a.region == 1)) return;
  }
  const bool own = (x0 < d.nx) && (j < d.ny);
  const long long PS = d.PS;
  const long long oc = (long long)(j + G) * d.PX + (x0 + G);
  const float* __restrict__ un = a.un;
  auto issue = [&](int s, int k, bool pf = false) {
    float* st = sm + s * L::SIZE;
    if (!pf) mbar_expect_tx(&bar[s], TX_BYTES);
    tma_ld(pf, st + L::U, &a.mun, &bar[s], i0, j0, k + GZ);
    tma_ld(pf, st + L::UP, &a.mup, &bar[s], i0 + G, j0 + G, k + GZ);
    tma_ld(pf, st + L::M, &a.mm, &bar[s], i0 + G, j0 + G, k + GZ);
    tma_ld(pf, st + L::UQ, &a.muq, &bar[s], i0 + G, j0 + G, k + 4 + GZ);
  };
  if (tid == 0) {
    for (int s = 0; s < ISO_NS; ++s) {
      mbar_init(&bar[s], 1);
      cnt[s] = 0u;
    }
    mbar_fence_init();
  }
  __syncthreads();
  if (tid == 0)
    for (int s = 0; s < ISO_NS && s < np; ++s) issue(s, k0 + s);
  if (tid == 0)
    for (int t = 0; t < L2PF && ISO_NS + t < np; ++t) issue(0, k0 + ISO_NS + t, true);

  // z-queue u^n(k-4 .. k+4); plane k+4 arrives with stage k (TMA)
  F4 q[9];
#pragma unroll
  for (int t = 0; t < 8; ++t) q[t] = ldg4(un + (long long)(k0 - 4 + t + GZ) * PS + oc);
  F4 exy{{0.f, 0.f, 0.f, 0.f}};
  F4 exv{{0.f, 0.f, 0.f, 0.f}};  // (SPML) eta_x dt per component
  float eyv = 0.f;               // (SPML) eta_y dt
  if (a.edx && own) {
    const F4 ex = ldg4(a.edx + x0);
    const float ey = a.edy[j];
#pragma unroll
    for (int e = 0; e < 4; ++e) exy.v[e] = ex.v[e] + ey;
    exv = ex;
    eyv = ey;
  }
  // (SPML) per-axis coefficients of this thread's points: x (4 points), y (its row)
  F4 cax{{2.f, 2.f, 2.f, 2.f}}, cbx{{1.f, 1.f, 1.f, 1.f}}, ccx{{1.f, 1.f, 1.f, 1.f}};
  float cay = 2.f, cby = 1.f, ccy = 1.f;
  if (SPML && a.spco[0] && own) {
    cax = ldg4(a.spco[0] + x0);
    cbx = ldg4(a.spco[0] + a.spnp[0] + x0);
    ccx = ldg4(a.spco[0] + 2 * a.spnp[0] + x0);
    cay = __ldg(a.spco[1] + j);
    cby = __ldg(a.spco[1] + a.spnp[1] + j);
    ccy = __ldg(a.spco[1] + 2 * a.spnp[1] + j);
  }
  const SrcHit sh = src_hit(a.src_o, oc, PS, 4);  // the source node of this column, if any
  // block-uniform: does this tile touch the x / y damping layer?  Planes outside the z layer
  // of such tiles take the undamped update without per-point branches (same arithmetic).
  const bool dxy = __syncthreads_or(exy.v[0] != 0.f || exy.v[1] != 0.f || exy.v[2] != 0.f || exy.v[3] != 0.f);

  // (SPML, SEIS_SPML_PF) this group's component indices at plane kk (-1: not a layer point)
  auto sp_index = [&](int kk, float ezk, int* six) {
#pragma unroll
    for (int e = 0; e < 4; ++e)
      six[e] = (own && x0 + e < d.nx && (exv.v[e] != 0.0f || eyv != 0.0f || ezk != 0.0f))
                   ? spml_idx(d, a.nbl, a.nxs, a.nys, exv.v[e], eyv, x0 + e, j, kk)
                   : -1;
  };
  float* const csl = sm + ISO_NS * L::SIZE + 4 * tid;  // [plane buffer][array][thread][4]
  constexpr int CST = NTX * BY * 4;
  // (the caller loads eta_z of plane kk one iteration earlier: no load latency at the issue)
  auto sp_issue = [&](int kk, int buf, float ezk) {  // cur (level n) arrays 0..2, nxt (n-1) 3..5
    if (dxy || ezk != 0.0f) {
      int six[4];
      sp_index(kk, ezk, six);
      const bool v = six[0] >= 0 && (six[0] & 3) == 0 && (a.spn & 3) == 0 && six[1] == six[0] + 1 &&
                     six[2] == six[0] + 2 && six[3] == six[0] + 3;
#pragma unroll
      for (int arr = 0; arr < 6; ++arr) {
        const float* src = a.sp + (long long)(arr < 3 ? a.lvl : 1 - a.lvl) * 3 * a.spn + (arr % 3) * a.spn;
        float* dst = csl + (buf * 6 + arr) * CST;
        if (v) {
          cp_async16(dst, src + six[0]);
        } else {
#pragma unroll
          for (int e = 0; e < 4; ++e)
            if (six[e] >= 0) cp_async4(dst + e, src + six[e], true);
        }
      }
    }
    cp_async_commit();  // (one group per plane, empty or not: uniform group counting)
  };
  auto ez_at = [&](int kk) { return (a.edx && kk < k1) ? __ldg(a.edz + kk + d.z0) : 0.0f; };
  float ez_pf = 0.0f;  // eta_z dt of plane k + 2 (loaded at iteration it - 1)
  if (SPML && SEIS_SPML_PF) {
    sp_issue(k0, 0, ez_at(k0));
    if (np > 1) sp_issue(k0 + 1, 1, ez_at(k0 + 1));
    else cp_async_commit();
    ez_pf = ez_at(k0 + 2);
  }

  SEIS_UNROLL(SEIS_ZU_ISO)
  for (int it = 0; it < np; ++it) {
    const int k = k0 + it;
    const int s = it % ISO_NS;
    const long long o = (long long)(k + GZ) * PS + oc;
    const float ez = a.edx ? a.edz[k + d.z0] : 0.0f;
    if (SPML && SEIS_SPML_PF) {
      if (it + 2 < np) sp_issue(k + 2, (it + 2) % 3, ez_pf);
      else cp_async_commit();
      ez_pf = ez_at(k + 3);
    }
    // (SPML) the layer components of this group are loaded before the stage wait (latency
    // overlap, as the C-PML memory variables): w0 = level n, wm = level n-1
    int sidx[4] = {-1, -1, -1, -1};
    float w0[3][4], wm[3][4];
    bool spv = false;  // the group's 4 components are one aligned float4 in every array
    if (SPML && (dxy || ez != 0.0f)) {
      sp_index(k, ez, sidx);
      spv = sidx[0] >= 0 && (sidx[0] & 3) == 0 && (a.spn & 3) == 0 && sidx[1] == sidx[0] + 1 &&
            sidx[2] == sidx[0] + 2 && sidx[3] == sidx[0] + 3;
      const float* cur = a.sp + (long long)a.lvl * 3 * a.spn;
      const float* nxt = a.sp + (long long)(1 - a.lvl) * 3 * a.spn;
      if (SEIS_SPML_PF) {  // (read after the stage wait, below)
      } else if (spv) {
#pragma unroll
        for (int c = 0; c < 3; ++c) {
          const F4 p0 = ld4(cur + c * a.spn + sidx[0]), pm = ld4(nxt + c * a.spn + sidx[0]);
#pragma unroll
          for (int e = 0; e < 4; ++e) {
            w0[c][e] = p0.v[e];
            wm[c][e] = pm.v[e];
          }
        }
      } else {
#pragma unroll
        for (int e = 0; e < 4; ++e)
          if (sidx[e] >= 0) {
#pragma unroll
            for (int c = 0; c < 3; ++c) {
              w0[c][e] = cur[c * a.spn + sidx[e]];
              wm[c][e] = nxt[c * a.spn + sidx[e]];
            }
          }
      }
    }
    if (SPML && SEIS_SPML_PSIPF > 0 && own && (tx & 7) == 0 && k + SEIS_SPML_PSIPF < k1) {
      const int kk = k + SEIS_SPML_PSIPF;
      const float ezk = a.edx ? __ldg(a.edz + kk + d.z0) : 0.0f;
      if (exv.v[0] != 0.0f || eyv != 0.0f || ezk != 0.0f) {
        const int ix = spml_idx(d, a.nbl, a.nxs, a.nys, exv.v[0], eyv, x0, j, kk);
#pragma unroll
        for (int c = 0; c < 6; ++c)
          prefetch_l2(a.sp + (long long)(c < 3 ? a.lvl : 1 - a.lvl) * 3 * a.spn + (c % 3) * a.spn + ix);
      }
    }
    mbar_wait(&bar[s], (it / ISO_NS) & 1);
    const float* st = sm + s * L::SIZE;
    q[8] = lds4(st + L::UQ + ty * TXV + 4 * tx);
    const float* c = st + L::U + (ty + 4) * W + 4 * tx + 4;  // u^n(x0, j, k)
    float xv[12];                                             // u^n(x0-4 .. x0+7, j)
    {
      const F4 a0 = lds4(c - 4), a1 = lds4(c), a2 = lds4(c + 4);
#pragma unroll
      for (int e = 0; e < 4; ++e) {
        xv[e] = a0.v[e];
        xv[4 + e] = a1.v[e];
        xv[8 + e] = a2.v[e];
      }
    }
    F4 ys[4];  // sum over the y pair (u_{j+m} + u_{j-m}), m = 1..4
#pragma unroll
    for (int m = 1; m <= 4; ++m) {
      const F4 yp = lds4(c + m * W), ym = lds4(c - m * W);
#pragma unroll
      for (int e = 0; e < 4; ++e) ys[m - 1].v[e] = yp.v[e] + ym.v[e];
    }
    const F4 upv = lds4(st + L::UP + ty * TXV + 4 * tx);
    const F4 mv = lds4(st + L::M + ty * TXV + 4 * tx);
    const bool damp = dxy || ez != 0.0f;
    float lap[4];
#pragma unroll
    for (int e = 0; e < 4; ++e) {
      float xs[4], yss[4], zs[4];
#pragma unroll
      for (int m = 0; m < 4; ++m) {
        xs[m] = xv[3 - m + e] + xv[5 + m + e];
        yss[m] = ys[m].v[e];
        zs[m] = q[3 - m].v[e] + q[5 + m].v[e];
      }
      lap[e] = iso_lap(xv[4 + e], xs, yss, zs);
    }
    F4 out;
    if (!damp) {  // block-uniform branch
#pragma unroll
      for (int e = 0; e < 4; ++e) out.v[e] = iso_update(xv[4 + e], upv.v[e], mv.v[e], lap[e], 0.0f);
    } else if (SPML) {
      // O6b: layer points advance u^(x), u^(y), u^(z), each damped along its own axis with the
      // 1D part L_d of the Laplacian; u^{n+1} is their sum.  Other points: Eq 1.
      if (SEIS_SPML_PF) {  // this plane's components, copied two planes ago
        cp_async_wait<2>();
        const float* cs = csl + (it % 3) * 6 * CST;
#pragma unroll
        for (int c = 0; c < 3; ++c) {
          const F4 p0 = lds4(cs + c * CST), pm = lds4(cs + (3 + c) * CST);
#pragma unroll
          for (int e = 0; e < 4; ++e) {
            w0[c][e] = p0.v[e];
            wm[c][e] = pm.v[e];
          }
        }
      }
#pragma unroll
      for (int e = 0; e < 4; ++e) {
        const float u = xv[4 + e];
        if (sidx[e] >= 0) {
          const int gz = k + d.z0;
          const float ca[3] = {cax.v[e], cay, __ldg(a.spco[2] + gz)};
          const float cb[3] = {cbx.v[e], cby, __ldg(a.spco[2] + a.spnp[2] + gz)};
          const float cc[3] = {ccx.v[e], ccy, __ldg(a.spco[2] + 2 * a.spnp[2] + gz)};
          float Ld[3];
          {
            float l = SEIS_C0 * u;
            l = fmaf(SEIS_C1, xv[3 + e] + xv[5 + e], l);
            l = fmaf(SEIS_C2, xv[2 + e] + xv[6 + e], l);
            l = fmaf(SEIS_C3, xv[1 + e] + xv[7 + e], l);
            Ld[0] = fmaf(SEIS_C4, xv[0 + e] + xv[8 + e], l);
            l = SEIS_C0 * u;
            l = fmaf(SEIS_C1, ys[0].v[e], l);
            l = fmaf(SEIS_C2, ys[1].v[e], l);
            l = fmaf(SEIS_C3, ys[2].v[e], l);
            Ld[1] = fmaf(SEIS_C4, ys[3].v[e], l);
            l = SEIS_C0 * u;
            l = fmaf(SEIS_C1, q[3].v[e] + q[5].v[e], l);
            l = fmaf(SEIS_C2, q[2].v[e] + q[6].v[e], l);
            l = fmaf(SEIS_C3, q[1].v[e] + q[7].v[e], l);
            Ld[2] = fmaf(SEIS_C4, q[0].v[e] + q[8].v[e], l);
          }
          float sum = 0.0f;
#pragma unroll
          for (int c = 0; c < 3; ++c) {
            // = [(2 - e^2) w0 - (1 - e) wm + m L_d] / (1 + e), e = eta_d dt (O6b)
            const float w1 = fmaf(ca[c], w0[c][e], fmaf(-cb[c], wm[c][e], cc[c] * (mv.v[e] * Ld[c])));
            wm[c][e] = w1;  // (the new level replaces n-1 in the same slot)
            sum += w1;
          }
          out.v[e] = sum;
        } else {
          out.v[e] = iso_update(u, upv.v[e], mv.v[e], lap[e], 0.0f);
        }
      }
      float* nxt = a.sp + (long long)(1 - a.lvl) * 3 * a.spn;
      if (spv) {
#pragma unroll
        for (int c = 0; c < 3; ++c) st4(nxt + c * a.spn + sidx[0], F4{{wm[c][0], wm[c][1], wm[c][2], wm[c][3]}});
      } else {
#pragma unroll
        for (int e = 0; e < 4; ++e)
          if (sidx[e] >= 0) {
#pragma unroll
            for (int c = 0; c < 3; ++c) nxt[c * a.spn + sidx[e]] = wm[c][e];
          }
      }
    } else {
#pragma unroll
      for (int e = 0; e < 4; ++e) {
        out.v[e] = iso_update(xv[4 + e], upv.v[e], mv.v[e], lap[e], exy.v[e] + ez);
      }
    }
    if (own) {
      if (sh.at(k)) {  // (selects, as ac_p)
        const float sa = a.src.get();
        const int se = sh.e();
#pragma unroll
        for (int e = 0; e < 4; ++e) {
          out.v[e] = (se == e) ? out.v[e] + sa : out.v[e];
          if (SPML && se == e && sidx[e] >= 0) a.sp[(long long)(1 - a.lvl) * 3 * a.spn + sidx[e]] += sa;  // x component
        }
      }
      st4_masked(a.up + o, out, x0, d.nx, true);
      if (GH) ghost_st4(a.gh, o, k, d.nzl, out, x0, d.nx);
      if (SNAP || IMG) {
        const long long cix = ((long long)k * d.ny + j) * d.nx + x0;
        const bool al = (d.nx & 3) == 0;
        if (SNAP) st4_masked(a.snap + cix, out, x0, d.nx, al);
        if (IMG) {
          F4 im;
#pragma unroll
          for (int e = 0; e < 4; ++e)
            im.v[e] = (x0 + e < d.nx) ? fmaf(a.imgR.at(cix + e), q[4].v[e], a.img[cix + e]) : 0.f;
          st4_masked(a.img + cix, im, x0, d.nx, false);
        }
      }
    }
    stage_release(&cnt[s], tid, it + ISO_NS < np, [&] {
      issue(s, k + ISO_NS);
      if (L2PF && it + ISO_NS + L2PF < np) issue(s, k + ISO_NS + L2PF, true);
    });
#pragma unroll
    for (int t = 0; t < 8; ++t) q[t] = q[t + 1];
  }
  if (SPML && SEIS_SPML_PF) cp_async_wait<0>();  // (no copy into this block's shared memory outlives it)
}

}  // namespace seis

// ------------------------------------------------------------------ small grids
// Persistent ISO modeling for L2-resident grids (C1, 64^3): the whole shot is ONE cooperative
// launch; every block owns fixed 4-point x-groups of the slab, and a grid-wide barrier
// separates the time steps (instead of two kernel launches per step: the grid is too small to
// hide launch gaps).  Per point it evaluates exactly the z-march kernel's expressions
// (iso_lap, iso_update, then the source add), so the results are bitwise the same.  Receiver
// gather of level n+1 (seis[n]) happens at the top of step n+1 (block 0 reads the input level,
// which that step does not write) and once after the last step.
#include <cooperative_groups.h>

namespace seis {

struct IsoPArgs {
  float* u0;                       // fld[0] / fld[1]: level n is u[cur], u^{n-1} / u^{n+1} u[1-cur]
  float* u1;
  const float* __restrict__ m;
  const float* __restrict__ edx;   // eta dt per axis (nullptr: no layer)
  const float* __restrict__ edy;
  const float* __restrict__ edz;
  Dims d;
  int nt, cur0;
  long long src_o;                 // padded source index (-1: none)
  const float* __restrict__ w;     // device wavelet [nt]; the amplitude is fmul_rn(src_scale, w[n])
  float src_scale;
  float* __restrict__ seis;        // [nt][nrec_tot]
  const long long* __restrict__ rec_off;
  const int* __restrict__ rec_id;
  int nrec, nrec_tot;
};

__global__ void __launch_bounds__(128) iso_persist_kernel(const __grid_constant__ IsoPArgs a) {
  namespace cg = cooperative_groups;
  cg::grid_group grid = cg::this_grid();
  const Dims& d = a.d;
  const int gx = (d.nx + 3) / 4;
  const long long ngroups = (long long)gx * d.ny * d.nzl;
  const long long PS = d.PS;
  int cur = a.cur0;
  for (int n = 0; n <= a.nt; ++n) {
    const float* __restrict__ un = cur ? a.u1 : a.u0;
    float* __restrict__ up = cur ? a.u0 : a.u1;
    if (n > 0 && blockIdx.x == 0)  // receivers of level n = seis[n - 1] (gather_kernel's rule)
      for (int r = threadIdx.x; r < a.nrec; r += blockDim.x)
        a.seis[(long long)(n - 1) * a.nrec_tot + a.rec_id[r]] = un[a.rec_off[r]];
    if (n == a.nt) break;
    for (long long g = blockIdx.x * (long long)blockDim.x + threadIdx.x; g < ngroups;
         g += (long long)gridDim.x * blockDim.x) {
      const int x0 = (int)(g % gx) * 4;
      const long long rest = g / gx;
      const int j = (int)(rest % d.ny), k = (int)(rest / d.ny);
      const long long o = d.at(x0, j, k);
      float xv[12];
      {
        const F4 a0 = ld4(un + o - 4), a1 = ld4(un + o), a2 = ld4(un + o + 4);
#pragma unroll
        for (int e = 0; e < 4; ++e) {
          xv[e] = a0.v[e];
          xv[4 + e] = a1.v[e];
          xv[8 + e] = a2.v[e];
        }
      }
      F4 yp[4], zp[4];
#pragma unroll
      for (int m = 1; m <= 4; ++m) {
        const F4 ya = ld4(un + o + m * d.PX), yb = ld4(un + o - m * d.PX);
        const F4 za = ld4(un + o - m * PS), zb = ld4(un + o + m * PS);
#pragma unroll
        for (int e = 0; e < 4; ++e) {
          yp[m - 1].v[e] = ya.v[e] + yb.v[e];
          zp[m - 1].v[e] = za.v[e] + zb.v[e];
        }
      }
      const F4 upv = ld4(up + o), mv = ldg4(a.m + o);
      F4 out;
#pragma unroll
      for (int e = 0; e < 4; ++e) {
        float xs[4], yss[4], zs[4];
#pragma unroll
        for (int m = 0; m < 4; ++m) {
          xs[m] = xv[3 - m + e] + xv[5 + m + e];
          yss[m] = yp[m].v[e];
          zs[m] = zp[m].v[e];
        }
        const float lap = iso_lap(xv[4 + e], xs, yss, zs);
        float eta = 0.0f;
        if (a.edx) eta = (__ldg(a.edx + x0 + e) + __ldg(a.edy + j)) + __ldg(a.edz + k + d.z0);
        out.v[e] = iso_update(xv[4 + e], upv.v[e], mv.v[e], lap, eta);
      }
      const long long rel = a.src_o - o;
      if (rel >= 0 && rel < 4) {
#pragma unroll
        for (int e = 0; e < 4; ++e)
          if (rel == e) out.v[e] += __fmul_rn(a.src_scale, __ldg(a.w + n));
      }
      st4_masked(up + o, out, x0, d.nx, true);
    }
    grid.sync();
    cur = 1 - cur;
  }
}


// ------------------------------------------------------------------ resident small-grid ISO
// iso_resident_kernel<TX>: the whole shot of a small ISO grid (nx <= 128) in one cooperative
// launch, each CTA OWNING one TX x 8 x 4 brick (TX = 64 or 128 >= nx: the whole x extent; the
// x halo is the zero ghost) for all nt steps.  u^{n-1}, m and eta of its points stay in
// registers, u^n of the brick + its 4-point halo (TX+8 x 16 x 12) in shared memory.
// Halo exchange without barriers or flags-then-data round trips (the low-latency protocol of
// NCCL's LL transport): every step the CTA writes its u^{n+1} into a per-brick exchange buffer
// as 8-byte (value, tag) pairs, tag = base + n + 1, with 16-byte relaxed stores; a neighbour
// polls the pairs it needs (y: 4 rows, z: the whole 4-plane brick) with relaxed 16-byte loads
// until both tags match -- an 8-byte pair is single-copy atomic, so a matching tag proves its
// value.  Two buffers per brick (step parity): a brick rewrites one only after consuming its
// neighbours' next step, which they wrote after consuming this one.  The 25-point star reads
// no corner values.  The field arrays receive the last two levels only (the final state).
// Per point it evaluates the z-march kernel's expressions in the same order (iso_lap,
// iso_update with eta = (eta_x + eta_y) + eta_z, then the source add fmul_rn(scale, w[n])),
// so it is bitwise equal to it (tests/test_persist_gpu.py).  Receiver values of level n
// (seis[n - 1]) are read from the tile centre at the top of step n and after the last step.
#ifndef SEIS_IR_NOWAIT
#define SEIS_IR_NOWAIT 0  // (perf-only builds: do not wait for the tags -- wrong results)
#endif
constexpr int IR_TY = 8, IR_TZ = 4, IR_H = IR_TY + 8, IR_D = IR_TZ + 8;
constexpr int IR_RECMAX = 1024;  // receivers of the shot (host-checked), hence per brick
template <int TX>
struct IrShape {
  static constexpr int W = TX + 8, TILE = W * IR_H * IR_D, OWN = TX * IR_TY * IR_TZ;
  static constexpr int GPT = TX <= 64 ? 1 : 2, THREADS = OWN / 4 / GPT;  // float4 groups per thread
  static constexpr int HALO = 3 * OWN / 2;                 // 16-byte (2-point) halo slots: z 2 x OWN/2, y 2 x OWN/4
  static constexpr int HPT = HALO / THREADS;               // per thread (12)
  static constexpr size_t smem() { return (size_t)(TILE + 2 * IR_RECMAX) * 4 + 128; }
  static_assert(HPT * THREADS == HALO && (OWN / 2) % THREADS == 0 && (OWN / 4) % THREADS == 0, "slots");
};
__device__ __forceinline__ void st_relaxed_v4(uint4* p, uint4 v) {
  asm volatile("st.relaxed.gpu.global.v4.u32 [%0], {%1, %2, %3, %4};" ::"l"(p), "r"(v.x), "r"(v.y), "r"(v.z),
               "r"(v.w)
               : "memory");
}
__device__ __forceinline__ uint4 ld_relaxed_v4(const uint4* p) {
  uint4 v;
  asm volatile("ld.relaxed.gpu.global.v4.u32 {%0, %1, %2, %3}, [%4];"
               : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w)
               : "l"(p)
               : "memory");
  return v;
}

struct IsoRArgs {
  float* u0;
  float* u1;
  const float* __restrict__ m;
  const float* __restrict__ edx;   // eta dt per axis (nullptr: no layer)
  const float* __restrict__ edy;
  const float* __restrict__ edz;
  Dims d;
  int nt, cur0;                    // (the shot starts from the zero state: u^0 = u^{-1} = 0)
  long long src_o;                 // padded source index (-1: none)
  const float* __restrict__ w;     // device wavelet [nt]; the amplitude is fmul_rn(src_scale, w[n])
  float src_scale;
  float* __restrict__ seis;        // [nt][nrec_tot]
  const long long* __restrict__ rec_off;
  const int* __restrict__ rec_id;
  int nrec, nrec_tot;
  uint4* xb;                       // [bricks][2][OWN / 2] exchange pairs (value, tag) x 2
  unsigned base;                   // tags of this shot: base + 1 .. base + nt (monotonic over shots)
  int nby, nbz;
  unsigned long long* trace;       // (SEIS_AS_TRACE builds) [brick][step][4] clock64 of thread 0
};

template <int TX>
__global__ void __launch_bounds__(IrShape<TX>::THREADS, 1)
    iso_resident_kernel(const __grid_constant__ IsoRArgs a) {
  using S = IrShape<TX>;
  constexpr int W = S::W, PL = W * IR_H, GPT = S::GPT, NT = S::THREADS, OWN = S::OWN;
  extern __shared__ __align__(128) float sm_raw[];
  float* tile = align128(sm_raw);
  int2* rl = reinterpret_cast<int2*>(tile + S::TILE);  // (receiver, tile index)
  __shared__ int nloc;
  const Dims& d = a.d;
  const int tid = threadIdx.x, b = blockIdx.x;
  const int by = b % a.nby, bz = b / a.nby;
  const int j0 = by * IR_TY, k0 = bz * IR_TZ;
  if (tid == 0) nloc = 0;
  for (int t = tid; t < S::TILE / 4; t += NT)  // u^0 = 0, and the zero x ghost
    reinterpret_cast<float4*>(tile)[t] = make_float4(0.f, 0.f, 0.f, 0.f);
  __syncthreads();
  for (int r = tid; r < a.nrec; r += NT) {  // this brick's receivers
    const long long off = a.rec_off[r];
    const int k = (int)(off / d.PS) - GZ;
    const long long rem = off % d.PS;
    const int j = (int)(rem / d.PX) - G, i = (int)(rem % d.PX) - G;
    if (j >= j0 && j < j0 + IR_TY && k >= k0 && k < k0 + IR_TZ) {
      const int e = atomicAdd(&nloc, 1);
      if (e < IR_RECMAX) rl[e] = make_int2(r, ((k - k0 + 4) * IR_H + (j - j0 + 4)) * W + i + 4);
    }
  }
  // halo slot t (16 bytes = 2 points): source pair in the exchange buffers (both parities
  // apart), tile destination; false: no neighbour on that side (the tile keeps the zero ghost)
  auto slot = [&](int t, int& src, int& dst) -> bool {
    int nb, e, rz, ry, x, row;
    if (t < OWN / 2) {  // z-: the neighbour's whole brick -> tile planes 0..3
      nb = bz > 0 ? b - a.nby : -1;
      e = 2 * t;
      rz = e / (IR_TY * TX), ry = (e / TX) % IR_TY, x = e % TX;
      src = e / 2;
      row = rz * IR_H + ry + 4;
    } else if (t < OWN) {  // z+: -> tile planes 8..11
      nb = bz + 1 < a.nbz ? b + a.nby : -1;
      e = 2 * (t - OWN / 2);
      rz = e / (IR_TY * TX), ry = (e / TX) % IR_TY, x = e % TX;
      src = e / 2;
      row = (rz + 4 + IR_TZ) * IR_H + ry + 4;
    } else {  // y- (its rows 4..7 -> tile rows 0..3) / y+ (its rows 0..3 -> tile rows 12..15)
      const bool lo = t < OWN + OWN / 4;
      nb = lo ? (by > 0 ? b - 1 : -1) : (by + 1 < a.nby ? b + 1 : -1);
      e = 2 * (t - (lo ? OWN : OWN + OWN / 4));
      rz = e / (4 * TX), ry = (e / TX) % 4, x = e % TX;
      src = ((rz * IR_TY + (lo ? 4 + ry : ry)) * TX + x) / 2;
      row = (rz + 4) * IR_H + (lo ? ry : 4 + IR_TY + ry);
    }
    dst = row * W + 4 + x;
    src += nb * 2 * (OWN / 2);
    return nb >= 0;
  };
  long long o[GPT];
  int cix[GPT], x0s[GPT];
  bool own[GPT];
  F4 upv[GPT], mv[GPT], eta[GPT];
#pragma unroll
  for (int q = 0; q < GPT; ++q) {
    const int g = tid + q * NT;
    const int x4 = g % (TX / 4), ry = (g / (TX / 4)) % IR_TY, rz = g / (TX / 4 * IR_TY);
    const int x0 = 4 * x4, j = j0 + ry, k = k0 + rz;
    x0s[q] = x0;
    own[q] = x0 < d.nx && j < d.ny && k < d.nzl;
    o[q] = d.at(x0, j, k);
    cix[q] = ((rz + 4) * IR_H + (ry + 4)) * W + 4 + x0;
    upv[q] = F4{{0.f, 0.f, 0.f, 0.f}};
    mv[q] = own[q] ? ldg4(a.m + o[q]) : F4{{0.f, 0.f, 0.f, 0.f}};
    eta[q] = F4{{0.f, 0.f, 0.f, 0.f}};
    if (a.edx && own[q]) {
      const F4 ex = ldg4(a.edx + x0);
      const float ey = a.edy[j], ez = a.edz[k + d.z0];
#pragma unroll
      for (int e = 0; e < 4; ++e) eta[q].v[e] = (ex.v[e] + ey) + ez;
    }
  }
  __syncthreads();  // (nloc)
  const int nl = min(nloc, IR_RECMAX);
  int cur = a.cur0;
  for (int n = 0; n < a.nt; ++n) {
    if (n > 0)  // receivers of level n (gather_kernel's rule: seis[n - 1])
      for (int e = tid; e < nl; e += NT) {
        const int2 rr = rl[e];
        a.seis[(long long)(n - 1) * a.nrec_tot + a.rec_id[rr.x]] = tile[rr.y];
      }
#if SEIS_AS_TRACE
    unsigned long long* tr = a.trace ? a.trace + ((size_t)b * a.nt + n) * 4 : nullptr;
    if (tr && tid == 0) tr[0] = clock64();
#endif
    const unsigned tag = a.base + (unsigned)n + 1u;
    const int par = (n + 1) & 1;
    uint4* xo = a.xb + ((size_t)b * 2 + par) * (OWN / 2);
    float* __restrict__ up = cur ? a.u0 : a.u1;  // u^{n-1} -> u^{n+1}
    F4 out[GPT];
#pragma unroll
    for (int q = 0; q < GPT; ++q) {
      const float* c = tile + cix[q];
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
      F4 ys[4], zs4[4];
#pragma unroll
      for (int m = 1; m <= 4; ++m) {
        const F4 yp = lds4(c + m * W), ym = lds4(c - m * W);
        const F4 zm = lds4(c - m * PL), zp = lds4(c + m * PL);
#pragma unroll
        for (int e = 0; e < 4; ++e) {
          ys[m - 1].v[e] = yp.v[e] + ym.v[e];
          zs4[m - 1].v[e] = zm.v[e] + zp.v[e];
        }
      }
#pragma unroll
      for (int e = 0; e < 4; ++e) {
        float xs[4], yss[4], zs[4];
#pragma unroll
        for (int m = 0; m < 4; ++m) {
          xs[m] = xv[3 - m + e] + xv[5 + m + e];
          yss[m] = ys[m].v[e];
          zs[m] = zs4[m].v[e];
        }
        const float lap = iso_lap(xv[4 + e], xs, yss, zs);
        out[q].v[e] = iso_update(xv[4 + e], upv[q].v[e], mv[q].v[e], lap, eta[q].v[e]);
      }
      if (own[q]) {
        const long long rel = a.src_o - o[q];
        if (rel >= 0 && rel < 4) {
#pragma unroll
          for (int e = 0; e < 4; ++e)
            if (rel == e) out[q].v[e] += __fmul_rn(a.src_scale, __ldg(a.w + n));
        }
        if (n + 2 >= a.nt) st4_masked(up + o[q], out[q], x0s[q], d.nx, true);  // the final state
      }
      // outside the domain: the zero ghost, for the tile and the neighbours
#pragma unroll
      for (int e = 0; e < 4; ++e)
        if (!own[q] || x0s[q] + e >= d.nx) out[q].v[e] = 0.f;
      const int g = tid + q * NT;
      st_relaxed_v4(xo + 2 * g, make_uint4(__float_as_uint(out[q].v[0]), tag, __float_as_uint(out[q].v[1]), tag));
      st_relaxed_v4(xo + 2 * g + 1, make_uint4(__float_as_uint(out[q].v[2]), tag, __float_as_uint(out[q].v[3]), tag));
#pragma unroll
      for (int e = 0; e < 4; ++e) upv[q].v[e] = xv[4 + e];  // u^n: the next step's u^{n-1}
    }
#if SEIS_AS_TRACE
    if (tr && tid == 0) tr[1] = clock64();
#endif
    __syncthreads();  // #1: the tile is consumed
#pragma unroll
    for (int q = 0; q < GPT; ++q)  // the brick's own u^{n+1} into the tile centre
      *reinterpret_cast<float4*>(tile + cix[q]) = make_float4(out[q].v[0], out[q].v[1], out[q].v[2], out[q].v[3]);
    {  // the neighbours' u^{n+1} halo pairs, in batches of HB 16-byte polls in flight
      const uint4* xi = a.xb + (size_t)par * (OWN / 2);
      constexpr int HB = S::HPT <= 6 ? S::HPT : S::HPT / 2;
#pragma unroll
      for (int h = 0; h < S::HPT; h += HB) {
        uint4 v[HB];
#pragma unroll
        for (int i = 0; i < HB; ++i) {
          int src, dst;
          if (slot(tid + (h + i) * NT, src, dst)) v[i] = ld_relaxed_v4(xi + src);
        }
#pragma unroll
        for (int i = 0; i < HB; ++i) {
          int src, dst;
          if (slot(tid + (h + i) * NT, src, dst)) {
            long long spins = 0;
            while (!SEIS_IR_NOWAIT && (v[i].y != tag || v[i].w != tag)) {
              if (++spins > (1ll << 24)) __trap();  // (a lost neighbour: fail, do not hang)
              v[i] = ld_relaxed_v4(xi + src);
            }
            *reinterpret_cast<float2*>(tile + dst) = make_float2(__uint_as_float(v[i].x), __uint_as_float(v[i].z));
          }
        }
      }
    }
#if SEIS_AS_TRACE
    if (tr && tid == 0) tr[2] = clock64();
#endif
    __syncthreads();  // #2: centre and halo of u^{n+1} are in the tile
#if SEIS_AS_TRACE
    if (tr && tid == 0) tr[3] = clock64();
#endif
    cur = 1 - cur;
  }
  for (int e = tid; e < nl; e += NT) {  // level nt
    const int2 rr = rl[e];
    a.seis[(long long)(a.nt - 1) * a.nrec_tot + a.rec_id[rr.x]] = tile[rr.y];
  }
}

}  // namespace seis
