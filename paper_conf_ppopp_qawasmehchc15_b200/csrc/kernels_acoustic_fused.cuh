// kernels_acoustic_fused.cuh — one full acoustic time step (Eq 2; V then P,
// O2/O8) in a single z-march (half-step temporal blocking).
//
// The split pair (kernels_acoustic.cuh) moves 56 B per point and step: V reads p, q, rho
// and writes q (32 B), P reads q, p, K and writes p (24 B).  Here one sweep reads
// p^n, q^{n-1/2}, rho, K and writes q^{n+1/2}, p^{n+1} once: 40 B per point (+ C-PML psi).
// The price is redundancy and double buffering:
//   * P at (x, y, k) needs q^{n+1/2} at x-4..x+3, y-4..y+3, k-4..k+3, values owned by the
//     neighbouring tiles / z-chunks, which may not have produced them yet.  Each block
//     therefore recomputes q_x on its 4-point x-halo groups and q_y on its 4-row y-halo
//     (in shared memory, never stored), and q_z three planes AHEAD of the march (plane k+3
//     at plane k, into a register queue; the 7 planes before a chunk are recomputed in its
//     warm-up).
//   * The recompute reads p^n, q^{n-1/2} and the V memory variables psi_p that other blocks
//     are updating -> the state is double-buffered: set `c` (read) -> set `1-c` (written);
//     psi_p likewise.  psi_q (P) is only ever touched by its owner and stays in place.
// Arithmetic per point is the split kernels' expression for expression, so results are
// bitwise identical to the split pair (tested).
//
// Block: 16 x BY threads, a 64 x BY (x, y) tile, 4 x-points per thread; one TMA stage per
// plane k (mbarrier ring, NS deep): the p^n tile with an 8-point x/y halo, the rho tile
// (x -4..71, y -4..BY+4), the old q_x (x halo 4) and q_y (y halo 4) tiles, and the 64 x BY
// tiles of q_z^{old}(k+3), rho(k+4), p^n(k+7) (z-queue feed) and dt K/h (k).  New q_x / q_y
// of plane k (tile + halos) go to a double-buffered shared tile that the P half reads after
// one __syncthreads per plane.
#pragma once
#include "common.cuh"
#include "kernels_acoustic.cuh"  // CpmlAxis

namespace seis {

#ifndef SEIS_AF_NS
#define SEIS_AF_NS 2
#endif
constexpr int AF_NS = SEIS_AF_NS;

struct AcFArgs {
  CUtensorMap mpt;   // p^n tile, box 80 x (BY+16), origin (i0-8, j0-8)
  CUtensorMap mrt;   // rho tile, box 76 x (BY+9), origin (i0-4, j0-4)
  CUtensorMap mqx;   // q_x^{old}, box 72 x BY, origin (i0-4, j0)
  CUtensorMap mqy;   // q_y^{old}, box 64 x (BY+8), origin (i0, j0-4)
  CUtensorMap mqz;   // q_z^{old}, box 64 x BY (plane k+3)
  CUtensorMap mrz;   // rho, box 64 x BY (plane k+4)
  CUtensorMap mpz;   // p^n, box 64 x BY (plane k+7)
  CUtensorMap mk;    // dt K / h, box 64 x BY (plane k)
  const float* __restrict__ p0;   // old set (read)
  const float* __restrict__ qz0;
  const float* __restrict__ rho;
  float* __restrict__ p1;         // new set (written)
  float* __restrict__ qx1;
  float* __restrict__ qy1;
  float* __restrict__ qz1;
  float dth;                      // dt / h
  int W, zlo;
  CpmlAxis cx, cy, cz;
  const float* __restrict__ psr[3];  // psi_{p,x|y|z} old (read)
  float* __restrict__ psw[3];        // psi_{p,x|y|z} new (written, own points)
  float* __restrict__ pq[3];         // psi_{q,x|y|z} (in place)
  Dims d;
  int zc;
  int ch0, chs;
  long long src_o;
  SrcAmp src;
  float* __restrict__ snap;
  const float* __restrict__ imgS;
  float* __restrict__ img;
};

template <int BY>
struct AcFStage {
  static constexpr int PW = TXV + 16, RW = TXV + 12, XW = TXV + 8, T = TXV * BY;
  static constexpr int PT = 0, RT = PT + PW * (BY + 16), QX = RT + ((RW * (BY + 9) + 31) / 32) * 32,
                       QY = QX + XW * BY, QZ = QY + TXV * (BY + 8), RZ = QZ + T, PZ = RZ + T, KK = PZ + T,
                       SIZE = KK + T;
  static constexpr uint32_t BYTES =
      (PW * (BY + 16) + RW * (BY + 9) + XW * BY + TXV * (BY + 8) + 4 * T) * 4;
  // double-buffered new q_x (72 x BY) / q_y (64 x (BY+8)) tiles
  static constexpr int NX = 0, NY = XW * BY, NSIZE = NY + TXV * (BY + 8);
  static constexpr size_t smem_bytes() { return ((size_t)AF_NS * SIZE + 2 * NSIZE) * 4 + 128; }
};

// staggered D+ at x+e+1/2 (e = 0..3) from 12 values v[0..11] = f(x-4 .. x+7)
__device__ __forceinline__ float dplus12(const float* v, int e) {
  float t = SEIS_D1 * (v[5 + e] - v[4 + e]);
  t = fmaf(SEIS_D2, v[6 + e] - v[3 + e], t);
  t = fmaf(SEIS_D3, v[7 + e] - v[2 + e], t);
  return fmaf(SEIS_D4, v[8 + e] - v[1 + e], t);
}
// staggered D- at x+e from 12 values v[0..11] = g(x-4 .. x+7)
__device__ __forceinline__ float dminus12(const float* v, int e) {
  float t = SEIS_D1 * (v[4 + e] - v[3 + e]);
  t = fmaf(SEIS_D2, v[5 + e] - v[2 + e], t);
  t = fmaf(SEIS_D3, v[6 + e] - v[1 + e], t);
  return fmaf(SEIS_D4, v[7 + e] - v[0 + e], t);
}
// D+ at the 1/2 point of a column window r[0..7] = f(c-3 .. c+4), component e
__device__ __forceinline__ float dplus_col(const F4* r, int e) {
  float t = SEIS_D1 * (r[4].v[e] - r[3].v[e]);
  t = fmaf(SEIS_D2, r[5].v[e] - r[2].v[e], t);
  t = fmaf(SEIS_D3, r[6].v[e] - r[1].v[e], t);
  return fmaf(SEIS_D4, r[7].v[e] - r[0].v[e], t);
}
// D- at c of a column window q[0..7] = g(c-4 .. c+3), component e
__device__ __forceinline__ float dminus_col(const F4* q, int e) {
  float t = SEIS_D1 * (q[4].v[e] - q[3].v[e]);
  t = fmaf(SEIS_D2, q[5].v[e] - q[2].v[e], t);
  t = fmaf(SEIS_D3, q[6].v[e] - q[1].v[e], t);
  return fmaf(SEIS_D4, q[7].v[e] - q[0].v[e], t);
}

template <int BY, bool SNAP, bool IMG>
__global__ void __launch_bounds__(NTX * BY, BY <= 16 ? 2 : 1) ac_fused_kernel(const __grid_constant__ AcFArgs a) {
  using L = AcFStage<BY>;
  constexpr int PW = L::PW, RW = L::RW, XW = L::XW;
  static_assert(L::RT % 32 == 0 && L::QX % 32 == 0 && L::QY % 32 == 0 && L::QZ % 32 == 0 &&
                    L::SIZE % 32 == 0 && L::NY % 32 == 0 && L::NSIZE % 32 == 0,
                "128-byte tiles");
  static_assert(NTX == 16, "4-point groups over a 64-wide tile");
  extern __shared__ __align__(128) float sm_raw[];
  float* sm = align128(sm_raw);
  float* qn = sm + AF_NS * L::SIZE;  // 2 x NSIZE
  __shared__ __align__(8) uint64_t bar[AF_NS];
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
  const int Wl = a.W;
  const float dth = a.dth;
  auto issue = [&](int s, int k, bool pf = false) {
    float* st = sm + s * L::SIZE;
    const int z = k + GZ, x = i0 + G, y = j0 + G;
    if (!pf) mbar_expect_tx(&bar[s], L::BYTES);
    tma_ld(pf, st + L::PT, &a.mpt, &bar[s], x - 8, y - 8, z);
    tma_ld(pf, st + L::RT, &a.mrt, &bar[s], x - 4, y - 4, z);
    tma_ld(pf, st + L::QX, &a.mqx, &bar[s], x - 4, y, z);
    tma_ld(pf, st + L::QY, &a.mqy, &bar[s], x, y - 4, z);
    tma_ld(pf, st + L::QZ, &a.mqz, &bar[s], x, y, z + 3);
    tma_ld(pf, st + L::RZ, &a.mrz, &bar[s], x, y, z + 4);
    tma_ld(pf, st + L::PZ, &a.mpz, &bar[s], x, y, z + 7);
    tma_ld(pf, st + L::KK, &a.mk, &bar[s], x, y, z);
  };
  if (tid == 0) {
    for (int s = 0; s < AF_NS; ++s) {
      mbar_init(&bar[s], 1);
    }
    mbar_fence_init();
  }
  __syncthreads();
  if (tid == 0)
    for (int s = 0; s < AF_NS && s < np; ++s) issue(s, k0 + s);
  if (tid == 0)
    for (int t = 0; t < L2PF && AF_NS + t < np; ++t) issue(0, k0 + AF_NS + t, true);

  const bool lxo = Wl > 0 && (x0 < Wl || x0 + 3 >= d.nx - Wl);  // own group may touch the x layer
  const bool lyo = Wl > 0 && CpmlIdx::in(j, d.ny, Wl, true);

  // ---- q_z^{n+1/2} at plane kq (local), own column: window pz[0..7] = p^n(kq-3 .. kq+4),
  // rho(kq), rho(kq+1); stores value (+ psi) when the plane belongs to this chunk.
  // psi_{p,z} old values of plane kq (loaded ahead of the TMA wait in the march)
  auto psz_in = [&](int kq) {
    const int gz = kq + d.z0;
    return own && Wl > 0 && gz >= 0 && gz < d.nz && CpmlIdx::in(gz, d.nz, Wl, a.zlo);
  };
  auto psz_base = [&](int kq) { return (CpmlIdx::slot(kq + d.z0, d.nz, Wl) * d.ny + j) * d.nx + x0; };
  auto psz_load = [&](int kq, float* o4) {
    if (psz_in(kq)) {
      const int base = psz_base(kq);
#pragma unroll
      for (int e = 0; e < 4; ++e) o4[e] = x0 + e < d.nx ? a.psr[2][base + e] : 0.f;
    }
  };
  auto qz_point = [&](const F4* pz, const F4& qold, const F4& r0, const F4& r1, int kq, bool store,
                      const float* pso) -> F4 {
    const int gz = kq + d.z0;
    F4 out{{0.f, 0.f, 0.f, 0.f}};
    if (!own || gz < 0 || gz >= d.nz) return out;  // outside the grid: ghost zeros (O1)
    float dz[4];
#pragma unroll
    for (int e = 0; e < 4; ++e) dz[e] = dplus_col(pz, e);
    if (psz_in(kq)) {
      const int base = psz_base(kq);
      const float za = __ldg(a.cz.ah + gz), zb = __ldg(a.cz.bh + gz);
#pragma unroll
      for (int e = 0; e < 4; ++e)
        if (x0 + e < d.nx) {
          const float v = fmaf(zb, pso[e], za * dz[e]);
          if (store) a.psw[2][base + e] = v;
          dz[e] += v;
        }
    }
    const bool zlast = gz + 1 >= d.nz;
#pragma unroll
    for (int e = 0; e < 4; ++e) {
      const float rzp = zlast ? r0.v[e] : r1.v[e];
      const float bz = dth * (2.0f * rcp_fast(r0.v[e] + rzp));
      out.v[e] = (x0 + e < d.nx) ? fmaf(bz, dz[e], qold.v[e]) : 0.f;
    }
    if (store) st4_masked(a.qz1 + (long long)(kq + GZ) * PS + oc, out, x0, d.nx, true);
    return out;
  };

  // ---- warm-up: p^n(k0-7 .. k0+6) window, q_z^{new}(k0-4 .. k0+2)
  F4 pz[8];   // p^n(k .. k+7) in the march (window of q_z(k+3))
  F4 qz[8];   // q_z^{new}(k-4 .. k+3)
  F4 rz3;     // rho(k+3)
  {
    const float* __restrict__ p0 = a.p0;
#pragma unroll
    for (int t = 0; t < 7; ++t) pz[t] = ldg4(p0 + (long long)(k0 - 7 + t + GZ) * PS + oc);
    F4 rlo = ldg4(a.rho + (long long)(k0 - 4 + GZ) * PS + oc);
#pragma unroll
    for (int t = 0; t < 7; ++t) {
      const int kq = k0 - 4 + t;
      pz[7] = ldg4(p0 + (long long)(kq + 4 + GZ) * PS + oc);
      const F4 rhi = ldg4(a.rho + (long long)(kq + 1 + GZ) * PS + oc);
      const F4 qo = ldg4(a.qz0 + (long long)(kq + GZ) * PS + oc);
      float pso[4];
      psz_load(kq, pso);
      qz[t] = qz_point(pz, qo, rlo, rhi, kq, kq >= k0 && kq < k1, pso);
      rlo = rhi;
#pragma unroll
      for (int u = 0; u < 7; ++u) pz[u] = pz[u + 1];
    }
    rz3 = rlo;  // rho(k0+3)
  }
  const long long srel0 = a.src_o - oc;

  for (int it = 0; it < np; ++it) {
    const int k = k0 + it;
    const int s = it % AF_NS;
    const long long o = (long long)(k + GZ) * PS + oc;
    const int gz = k + d.z0;
    float* qnx = qn + (it & 1) * L::NSIZE + L::NX;
    float* qny = qn + (it & 1) * L::NSIZE + L::NY;
    // C-PML psi_q (P, in place) old values before the wait; 32-bit compact-slab indices
    // (recomputed for the store: fewer live registers across the V half)
    const bool lz = Wl > 0 && CpmlIdx::in(gz, d.nz, Wl, a.zlo);
    auto ixq = [&](int e) {  // x-slab index of point x0 + e, -1 outside the layer
      const int x = x0 + e;
      return (x < d.nx && CpmlIdx::in(x, d.nx, Wl, true)) ? (k * d.ny + j) * (2 * Wl) + CpmlIdx::slot(x, d.nx, Wl)
                                                          : -1;
    };
    const int iyq = lyo ? (k * (2 * Wl) + CpmlIdx::slot(j, d.ny, Wl)) * d.nx + x0 : 0;
    const int izq = lz ? (CpmlIdx::slot(gz, d.nz, Wl) * d.ny + j) * d.nx + x0 : 0;
    float ox[4], oy[4], oz[4], ozp[4];
    psz_load(k + 3, ozp);
    if (own && lxo) {
#pragma unroll
      for (int e = 0; e < 4; ++e) {
        const int i = ixq(e);
        ox[e] = i >= 0 ? a.pq[0][i] : 0.f;
      }
    }
    if (own && lyo) {
#pragma unroll
      for (int e = 0; e < 4; ++e) oy[e] = x0 + e < d.nx ? a.pq[1][iyq + e] : 0.f;
    }
    if (own && lz) {
#pragma unroll
      for (int e = 0; e < 4; ++e) oz[e] = x0 + e < d.nx ? a.pq[2][izq + e] : 0.f;
    }
    mbar_wait(&bar[s], (it / AF_NS) & 1);
    const float* st = sm + s * L::SIZE;
    const int pt = ty * TXV + 4 * tx;
    // ---- V, z component, plane k+3
    pz[7] = lds4(st + L::PZ + pt);
    {
      const F4 r4 = lds4(st + L::RZ + pt);
      const F4 qo = lds4(st + L::QZ + pt);
      qz[7] = qz_point(pz, qo, rz3, r4, k + 3, k + 3 < k1, ozp);
      rz3 = r4;
    }
    // ---- V, x component at group xg (row r of the tile), plane k -> shared (and HBM if own)
    auto vx = [&](int xg, int r, float* dst, bool store) {
      const int jr = j0 + r;
      const float* pr = st + L::PT + (r + 8) * PW + (xg - i0 + 8);
      float xv[12];
      {
        const F4 a0 = lds4(pr - 4), a1 = lds4(pr), a2 = lds4(pr + 4);
#pragma unroll
        for (int e = 0; e < 4; ++e) {
          xv[e] = a0.v[e];
          xv[4 + e] = a1.v[e];
          xv[8 + e] = a2.v[e];
        }
      }
      float dx[4];
#pragma unroll
      for (int e = 0; e < 4; ++e) dx[e] = dplus12(xv, e);
      const bool in = jr < d.ny && xg >= 0 && xg < d.nx;
      if (in && Wl > 0 && (xg < Wl || xg + 3 >= d.nx - Wl)) {
        int ix[4];
        psi_idx_x<4>(ix, d, Wl, xg, jr, k);
#pragma unroll
        for (int e = 0; e < 4; ++e)
          if (ix[e] >= 0) {
            const int x = xg + e;
            const float v = fmaf(__ldg(a.cx.bh + x), a.psr[0][ix[e]], __ldg(a.cx.ah + x) * dx[e]);
            if (store) a.psw[0][ix[e]] = v;
            dx[e] += v;
          }
      }
      const float* rc = st + L::RT + (r + 4) * RW + (xg - i0 + 4);
      const F4 r0 = lds4(rc);
      const float rx5 = rc[4];
      const F4 qo = lds4(st + L::QX + r * XW + (xg - i0 + 4));
      F4 out;
#pragma unroll
      for (int e = 0; e < 4; ++e) {
        const float rxp = (xg + e + 1 < d.nx) ? (e < 3 ? r0.v[e + 1] : rx5) : r0.v[e];
        const float bx = dth * (2.0f * rcp_fast(r0.v[e] + rxp));
        out.v[e] = (in && xg + e < d.nx) ? fmaf(bx, dx[e], qo.v[e]) : 0.f;
      }
      *reinterpret_cast<float4*>(dst) = make_float4(out.v[0], out.v[1], out.v[2], out.v[3]);
      if (store && in) st4_masked(a.qx1 + o + (long long)(r - ty) * d.PX + (xg - x0), out, xg, d.nx, true);
    };
    // ---- V, y component at column group g (x = i0 + 4g), tile row r (-4 .. BY+3), plane k
    auto vy = [&](int g, int r, float* dst, bool store) {
      const int jr = j0 + r, xg = i0 + 4 * g;
      const float* pc = st + L::PT + (r + 8) * PW + (4 * g + 8);
      F4 yr[8];
#pragma unroll
      for (int m = 0; m < 8; ++m) yr[m] = lds4(pc + (m - 3) * PW);
      float dy[4];
#pragma unroll
      for (int e = 0; e < 4; ++e) dy[e] = dplus_col(yr, e);
      const bool in = jr >= 0 && jr < d.ny && xg < d.nx;
      if (in && Wl > 0 && CpmlIdx::in(jr, d.ny, Wl, true)) {
        const long long base = ((long long)k * (2 * Wl) + CpmlIdx::slot(jr, d.ny, Wl)) * d.nx + xg;
        const float ya = __ldg(a.cy.ah + jr), yb = __ldg(a.cy.bh + jr);
#pragma unroll
        for (int e = 0; e < 4; ++e)
          if (xg + e < d.nx) {
            const float v = fmaf(yb, a.psr[1][base + e], ya * dy[e]);
            if (store) a.psw[1][base + e] = v;
            dy[e] += v;
          }
      }
      const float* rc = st + L::RT + (r + 4) * RW + (4 * g + 4);
      const F4 r0 = lds4(rc), ryn = lds4(rc + RW);
      const F4 qo = lds4(st + L::QY + (r + 4) * TXV + 4 * g);
      F4 out;
#pragma unroll
      for (int e = 0; e < 4; ++e) {
        const float ryp = (jr + 1 < d.ny) ? ryn.v[e] : r0.v[e];
        const float by = dth * (2.0f * rcp_fast(r0.v[e] + ryp));
        out.v[e] = (in && xg + e < d.nx) ? fmaf(by, dy[e], qo.v[e]) : 0.f;
      }
      *reinterpret_cast<float4*>(dst) = make_float4(out.v[0], out.v[1], out.v[2], out.v[3]);
      if (store && in) st4_masked(a.qy1 + o, out, xg, d.nx, true);
    };
    vx(x0, ty, qnx + ty * XW + 4 * tx + 4, true);
    vy(tx, ty, qny + (ty + 4) * TXV + 4 * tx, true);
    // halo groups: the first 2 BY threads (whole warps) the two x-halo groups of every row, the
    // next 4 warps the y-halo rows
    if (tid < 2 * BY) {
      const int r = tid >> 1, side = tid & 1;
      vx(side ? i0 + TXV : i0 - 4, r, qnx + r * XW + (side ? TXV + 4 : 0), false);
    } else if (tid >= 2 * BY && tid < 2 * BY + 8 * NTX) {
      const int t = tid - 2 * BY, rr = t / NTX, g = t % NTX;
      const int r = rr < 4 ? rr - 4 : BY + rr - 4;
      vy(g, r, qny + (r + 4) * TXV + 4 * g, false);
    }
    const F4 kv = lds4(st + L::KK + pt);
    if (IMG && own) {
      const long long cix = ((long long)k * d.ny + j) * d.nx + x0;
      F4 im;
#pragma unroll
      for (int e = 0; e < 4; ++e)
        im.v[e] = (x0 + e < d.nx) ? fmaf(__ldg(a.imgS + cix + e), pz[0].v[e], a.img[cix + e]) : 0.f;
      st4_masked(a.img + cix, im, x0, d.nx, false);
    }
    // all reads of stage s and all writes of the new q_x / q_y tiles are done
    __syncthreads();
    if (tid == 0 && it + AF_NS < np) {
      fence_proxy_async();
      issue(s, k + AF_NS);
      if (L2PF && it + AF_NS + L2PF < np) issue(s, k + AF_NS + L2PF, true);
    }
    // ---- P at plane k
    if (own) {
      float xv[12];
      {
        const float* c = qnx + ty * XW + 4 * tx + 4;
        const F4 a0 = lds4(c - 4), a1 = lds4(c), a2 = lds4(c + 4);
#pragma unroll
        for (int e = 0; e < 4; ++e) {
          xv[e] = a0.v[e];
          xv[4 + e] = a1.v[e];
          xv[8 + e] = a2.v[e];
        }
      }
      F4 yr[8];
      {
        const float* c = qny + (ty + 4) * TXV + 4 * tx;
#pragma unroll
        for (int m = 0; m < 8; ++m) yr[m] = lds4(c + (m - 4) * TXV);
      }
      float dx[4], dy[4], dz[4];
#pragma unroll
      for (int e = 0; e < 4; ++e) {
        dx[e] = dminus12(xv, e);
        dy[e] = dminus_col(yr, e);
        dz[e] = dminus_col(qz, e);
      }
      if (lxo) {
#pragma unroll
        for (int e = 0; e < 4; ++e) {
          const int i = ixq(e);
          if (i >= 0) {
            const int x = x0 + e;
            const float v = fmaf(__ldg(a.cx.b + x), ox[e], __ldg(a.cx.a + x) * dx[e]);
            a.pq[0][i] = v;
            dx[e] += v;
          }
        }
      }
      if (lyo) {
        const float ya = __ldg(a.cy.a + j), yb = __ldg(a.cy.b + j);
#pragma unroll
        for (int e = 0; e < 4; ++e)
          if (x0 + e < d.nx) {
            const float v = fmaf(yb, oy[e], ya * dy[e]);
            a.pq[1][iyq + e] = v;
            dy[e] += v;
          }
      }
      if (lz) {
        const float za = __ldg(a.cz.a + gz), zb = __ldg(a.cz.b + gz);
#pragma unroll
        for (int e = 0; e < 4; ++e)
          if (x0 + e < d.nx) {
            const float v = fmaf(zb, oz[e], za * dz[e]);
            a.pq[2][izq + e] = v;
            dz[e] += v;
          }
      }
      F4 out;
#pragma unroll
      for (int e = 0; e < 4; ++e) out.v[e] = fmaf(kv.v[e], (dx[e] + dy[e]) + dz[e], pz[0].v[e]);
      const long long rel = srel0 - (long long)(k + GZ) * PS;
      if (rel >= 0 && rel < 4) {
#pragma unroll
        for (int e = 0; e < 4; ++e)
          if (rel == e) out.v[e] += a.src.get();
      }
      st4_masked(a.p1 + o, out, x0, d.nx, true);
      if (SNAP) st4_masked(a.snap + ((long long)k * d.ny + j) * d.nx + x0, out, x0, d.nx, (d.nx & 3) == 0);
    }
#pragma unroll
    for (int t = 0; t < 7; ++t) {
      pz[t] = pz[t + 1];
      qz[t] = qz[t + 1];
    }
  }
}

}  // namespace seis
