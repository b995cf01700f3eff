// kernels_iso2.cuh — two ISO time steps (Eq 1) in ONE persistent launch: 2-step
// temporal blocking ("2-step temporal blocking for ISO (16 -> ~10 B/pt-step)").
//
// The one-step z-march (kernels_iso.cuh) moves 16 B per point and step: read u^n, u^{n-1}, m,
// write u^{n+1}.  Two steps in one sweep read u^n, u^{n-1}, m once and write u^{n+1}, u^{n+2}:
// 20 B per two steps.  Step 2 at (x, y, k) needs u^{n+1} on x-4..x+4, y-4..y+4 (in-plane) and
// k-4..k+4 (own column), i.e. values of the neighbouring tiles; as in the fused acoustic step
// (kernels_acoustic_step.cuh) the tiles exchange them through L2 as a wavefront instead of
// recomputing halos:
//
//   * one CTA per (128 x TY) xy tile, all tiles co-resident (cooperative launch, one CTA per
//     SM), each marching the whole z range: at iteration j it runs step 1 at plane j, then
//     step 2 at plane k = j - 4, IN PLACE: u^{n+1} over u^{n-1} (array B), u^{n+2} over u^n
//     (array A);
//   * step 2 at plane k needs u^{n+1}(k) of the x / y neighbour tiles: once every consumer warp
//     has arrived on the stage of step 1 (k) (after its stores), the producer thread publishes
//     the plane with a release add on the tile's counter; the step-2 producer acquires the own
//     + 4 neighbour counters >= k + 1 before it TMA-loads the u^{n+1} tile (+ halo 4) of plane k;
//   * the overwrite of u^n(k) by u^{n+2}(k) is safe: the only foreign readers of u^n(k) are the
//     neighbours' step 1 (k) halo loads, complete before their counters passed k; the own
//     column of u^n is read from a register queue (the z-feed of plane j + 4 happens 8 planes
//     before step 2 overwrites it);
//   * u^n (k - 4 .. k + 4 around step 1) and u^{n+1} (around step 2) live in 9-deep register
//     queues; step 2 reads its previous level u^n(k) from the first queue's oldest entry.
//
// The damped-wave layer (O6) has no memory variables: layer tiles move the same bytes as the
// others, so the lockstep wavefront is balanced (the acoustic C-PML imbalance of DESIGN §6
// does not arise).  Per point the arithmetic is the one-step kernel's expression for
// expression (iso_lap, iso_update with eta = (eta_x + eta_y) + eta_z, then the source add),
// so two launches of iso_step and one of this kernel are bitwise identical (tested).
// Forward modeling without snapshots / imaging, one slab, one process; the runtime falls back
// to the one-step kernel elsewhere and for a trailing odd step.
//
// Measured (B200, 512^3, nb = 20; profiles/r02_iso2.log, r02_iso2_ncu_summary.txt): 0.892 ms
// per launch of two steps (46 % of HBM at 20 B per point) against 2 x 0.353 ms for the
// one-step kernel (93 % at 16 B): the ISO update is issue-heavy (the one-step kernel is 72 %
// issue-active at 20 warps per SM), and one CTA of 14 consumer warps per SM -- 128 registers
// with the two 9-deep float4 queues -- hides less latency (60 % issue-active, short-scoreboard
// stalls on the shared tiles lead).  Deeper rings are slower (4 / 4 stages 1.27 ms).  So the
// kernel is opt-in (SEIS_ISO2=1), not the default.
#pragma once
#include "common.cuh"
#include "kernels_iso.cuh"  // iso_lap, iso_update

namespace seis {

#ifndef SEIS_I2_TY
#define SEIS_I2_TY 14
#endif
constexpr int I2_TX = 128;
constexpr int I2_TY = SEIS_I2_TY;
constexpr int I2_NTX = I2_TX / 4;          // consumer threads per row (4 x-points each)
constexpr int I2_CONS = I2_NTX * I2_TY;    // consumer threads
constexpr int I2_CWARPS = I2_CONS / 32;    // consumer warps (= empty-barrier arrivals per stage)
constexpr int I2_THREADS = I2_CONS + 64;   // + two producer warps (step-1 loads, step-2 loads)
constexpr int I2_L = 4;                    // step 2 lags step 1 by 4 planes
#ifndef SEIS_I2_NS1
#define SEIS_I2_NS1 3
#endif
#ifndef SEIS_I2_NS2
#define SEIS_I2_NS2 3
#endif
constexpr int I2_NS1 = SEIS_I2_NS1, I2_NS2 = SEIS_I2_NS2;

struct Iso2Args {
  CUtensorMap mat;   // u^n (A), box (128+8) x (TY+8), origin (i0-4, j0-4)       (step 1)
  CUtensorMap mbc;   // u^{n-1} (B), box 128 x TY                                   (step 1)
  CUtensorMap mm;    // m, box 128 x TY                                             (steps 1, 2)
  CUtensorMap mac;   // u^n (A), box 128 x TY (plane j + 4: the z-queue feed)       (step 1)
  CUtensorMap mbt;   // u^{n+1} (B), box (128+8) x (TY+8)                            (step 2)
  const float* ua;   // A = u^n -> u^{n+2} (padded)
  float* ub;         // B = u^{n-1} -> u^{n+1}
  float* uaw;        // A again (stores of step 2)
  const float* __restrict__ edx;  // eta dt per axis (nullptr: no layer)
  const float* __restrict__ edy;
  const float* __restrict__ edz;
  Dims d;
  int ntx, nty;               // tiles (gridDim.x = ntx * nty)
  unsigned* __restrict__ cnt; // per-tile step-1 progress counters (zeroed before the launch)
  long long src_o;            // padded source index in this slab, -1 = none
  SrcAmp src1, src2;          // amplitudes of steps n and n + 1
};

struct Iso2Layout {
  static constexpr int W = I2_TX + 8, H = I2_TY + 8, T = I2_TX * I2_TY;
  // step-1 stage: u^n tile + halo, u^{n-1}, m, u^n feed (plane j + 4)
  static constexpr int A = 0, B = A + r32(W * H), M = B + r32(T), F = M + r32(T), S1 = F + r32(T);
  static constexpr uint32_t S1BYTES = (W * H + 3 * T) * 4;
  // step-2 stage: u^{n+1} tile + halo, m
  static constexpr int U1 = 0, M2 = U1 + r32(W * H), S2 = M2 + r32(T);
  static constexpr uint32_t S2BYTES = (W * H + T) * 4;
  static constexpr size_t smem_bytes() { return ((size_t)I2_NS1 * S1 + (size_t)I2_NS2 * S2) * 4 + 128; }
};

template <bool DAMP>
__global__ void __launch_bounds__(I2_THREADS, 1) iso2_kernel(const __grid_constant__ Iso2Args a) {
  using L = Iso2Layout;
  constexpr int W = L::W;
  static_assert(L::B % 32 == 0 && L::M % 32 == 0 && L::F % 32 == 0 && L::S1 % 32 == 0 && L::M2 % 32 == 0 &&
                    L::S2 % 32 == 0,
                "128-byte tiles");
  extern __shared__ __align__(128) float sm_raw[];
  float* sm = align128(sm_raw);
  float* sm1 = sm;                      // I2_NS1 step-1 stages
  float* sm2 = sm + I2_NS1 * L::S1;     // I2_NS2 step-2 stages
  __shared__ __align__(8) uint64_t full1[I2_NS1], empty1[I2_NS1], full2[I2_NS2], empty2[I2_NS2];
  const Dims& d = a.d;
  const int tid = threadIdx.x;
  const int tile = blockIdx.x;
  const int tix = tile % a.ntx, tiy = tile / a.ntx;
  const int i0 = tix * I2_TX, j0 = tiy * I2_TY;
  const int nz = d.nzl;
  if (tid == 0) {
    for (int s = 0; s < I2_NS1; ++s) {
      mbar_init(&full1[s], 1);
      mbar_init(&empty1[s], I2_CWARPS);
    }
    for (int s = 0; s < I2_NS2; ++s) {
      mbar_init(&full2[s], 1);
      mbar_init(&empty2[s], I2_CWARPS);
    }
    mbar_fence_init();
  }
  __syncthreads();

  if (tid >= I2_CONS) {
    // ---------------------------------------------------------------- producer warps (lane 0)
    const int pw = (tid - I2_CONS) >> 5, lane = tid & 31;
    const int x = i0 + G, y = j0 + G;
    if (pw == 0 && lane == 0) {
      // step-1 stages: a free slot only.  The slot of plane j - NS1 is free again when all
      // consumer warps arrived on it, i.e. after step 1 (j - NS1) INCLUDING its u^{n+1} stores:
      // then the plane is published to the neighbour tiles (release add on the tile counter).
      unsigned* const mycnt = a.cnt + tile;
      for (int j = 0; j < nz + I2_NS1; ++j) {
        const int s = j % I2_NS1;
        if (j >= I2_NS1) {
          mbar_wait_nap(&empty1[s], ((j / I2_NS1) - 1) & 1);
          fence_proxy_async_global();
          red_release_gpu_add(mycnt, 1u);
        }
        if (j >= nz) continue;
        float* st = sm1 + s * L::S1;
        const int z = j + GZ;
        mbar_expect_tx(&full1[s], L::S1BYTES);
        tma_load_3d(st + L::A, &a.mat, &full1[s], i0, j0, z);
        tma_load_3d(st + L::B, &a.mbc, &full1[s], x, y, z);
        tma_load_3d(st + L::M, &a.mm, &full1[s], x, y, z);
        tma_load_3d(st + L::F, &a.mac, &full1[s], x, y, z + 4);
      }
    } else if (pw == 1 && lane == 0) {
      // step-2 stages: a free slot, then step 1 (k) complete in this tile and its x / y
      // neighbours (acquire loads of their counters), then the u^{n+1} tile (+ halo) and m.
      const unsigned* cs[5] = {a.cnt + tile, tix > 0 ? a.cnt + tile - 1 : nullptr,
                               tix + 1 < a.ntx ? a.cnt + tile + 1 : nullptr,
                               tiy > 0 ? a.cnt + tile - a.ntx : nullptr,
                               tiy + 1 < a.nty ? a.cnt + tile + a.ntx : nullptr};
      unsigned seen[5] = {0u, 0u, 0u, 0u, 0u};
      for (int k = 0; k < nz; ++k) {
        const int s = k % I2_NS2;
        if (k >= I2_NS2) mbar_wait_nap(&empty2[s], ((k / I2_NS2) - 1) & 1);
        const unsigned need = (unsigned)(k + 1);
        for (;;) {
          bool ok = true;
#pragma unroll
          for (int c = 0; c < 5; ++c)
            if (cs[c] && seen[c] < need) seen[c] = ld_relaxed_gpu(cs[c]);
#pragma unroll
          for (int c = 0; c < 5; ++c) ok = ok && (!cs[c] || seen[c] >= need);
          if (ok) break;
          __nanosleep(SEIS_AS_NAP);
        }
        fence_acq_rel_gpu();         // acquire: the u^{n+1} stores released with the counters
        fence_proxy_async_global();  // ... ordered before the TMA (async proxy) reads
        float* st = sm2 + s * L::S2;
        const int z = k + GZ;
        mbar_expect_tx(&full2[s], L::S2BYTES);
        tma_load_3d(st + L::U1, &a.mbt, &full2[s], i0, j0, z);
        tma_load_3d(st + L::M2, &a.mm, &full2[s], x, y, z);
      }
    }
    return;
  }

  // ------------------------------------------------------------------ consumer threads
  const int tx = tid % I2_NTX, ty = tid / I2_NTX;
  const int x0 = i0 + 4 * tx, jy = j0 + ty;
  const bool own = (x0 < d.nx) && (jy < d.ny);
  const long long PS = d.PS;
  const long long oc = (long long)(jy + G) * d.PX + (x0 + G);
  const int lane = tid & 31;
  const int pt = ty * I2_TX + 4 * tx;
  // eta_x + eta_y of this thread's points (the damped-wave layer, O6)
  F4 exy{{0.f, 0.f, 0.f, 0.f}};
  if (DAMP && own) {
    const F4 ex = ldg4(a.edx + x0);
    const float ey = a.edy[jy];
#pragma unroll
    for (int e = 0; e < 4; ++e) exy.v[e] = ex.v[e] + ey;
  }
  const long long srel0 = a.src_o - oc;
  // z-queues: r = u^n(j-4 .. j+4) at step 1 (j) (plane j + 4 arrives with the stage);
  // q = u^{n+1}(j-8 .. j) after step 1 (j) appended, i.e. (k-4 .. k+4) for step 2 (k = j - 4)
  F4 r[9], q[9];
#pragma unroll
  for (int t = 0; t < 8; ++t) r[t] = ldg4(a.ua + (long long)(t - 4 + GZ) * PS + oc);
#pragma unroll
  for (int t = 0; t < 9; ++t) q[t] = F4{{0.f, 0.f, 0.f, 0.f}};

  // one step at plane kk from the centre pointer c (tile row of the point, x-halo 4, row
  // stride W), the z-queue zq (9 planes), the previous level upv and m
  auto one = [&](const float* c, const F4* zq, const F4& upv, const F4& mv, int kk) {
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
    F4 ys[4];  // (u_{j+m} + u_{j-m}), m = 1..4 (the one-step kernel's pair order)
#pragma unroll
    for (int m = 1; m <= 4; ++m) {
      const F4 yp = lds4(c + m * W), ym = lds4(c - m * W);
#pragma unroll
      for (int e = 0; e < 4; ++e) ys[m - 1].v[e] = yp.v[e] + ym.v[e];
    }
    const float ez = DAMP ? __ldg(a.edz + kk + d.z0) : 0.0f;
    F4 out;
#pragma unroll
    for (int e = 0; e < 4; ++e) {
      float xs[4], yss[4], zs[4];
#pragma unroll
      for (int m = 0; m < 4; ++m) {
        xs[m] = xv[3 - m + e] + xv[5 + m + e];
        yss[m] = ys[m].v[e];
        zs[m] = zq[3 - m].v[e] + zq[5 + m].v[e];
      }
      const float lap = iso_lap(xv[4 + e], xs, yss, zs);
      out.v[e] = iso_update(xv[4 + e], upv.v[e], mv.v[e], lap, DAMP ? exy.v[e] + ez : 0.0f);
    }
    return out;
  };

  for (int j = 0; j < nz + I2_L; ++j) {
    // ================================ step 1 at plane j: u^{n+1}(j) into B
    F4 u1{{0.f, 0.f, 0.f, 0.f}};  // (planes >= nz: the zero ghost)
    if (j < nz) {
      const int s = j % I2_NS1;
      mbar_wait(&full1[s], (j / I2_NS1) & 1);
      const float* st = sm1 + s * L::S1;
      r[8] = lds4(st + L::F + pt);
      const F4 upv = lds4(st + L::B + pt), mv = lds4(st + L::M + pt);
      const float* c = st + L::A + (ty + 4) * W + 4 * tx + 4;  // u^n(x0, jy, j)
      F4 out = one(c, r, upv, mv, j);
      __syncwarp();
      if (own) {
        const long long rel = srel0 - (long long)(j + GZ) * PS;
        if (rel >= 0 && rel < 4) {
#pragma unroll
          for (int e = 0; e < 4; ++e)
            if (rel == e) out.v[e] += a.src1.get();
        }
        st4_masked(a.ub + (long long)(j + GZ) * PS + oc, out, x0, d.nx, true);
#pragma unroll
        for (int e = 0; e < 4; ++e)
          if (x0 + e >= d.nx) out.v[e] = 0.f;  // (outside the grid: the zero ghost)
        u1 = out;
      }
      // release the stage after this warp's stores: the producer publishes step 1 (j) of the
      // tile once all warps arrived
      __syncwarp();
      if (lane == 0) mbar_arrive(&empty1[s]);
    }
    // u^{n+1} queue: append plane j (q[8]); u^n(j - 4) = r[0] is step 2's previous level
#pragma unroll
    for (int t = 0; t < 8; ++t) q[t] = q[t + 1];
    q[8] = u1;
    if (j >= I2_L) {
      // ================================ step 2 at plane k = j - 4: u^{n+2}(k) into A
      const int k = j - I2_L;
      const int s = k % I2_NS2;
      mbar_wait(&full2[s], (k / I2_NS2) & 1);
      const float* st = sm2 + s * L::S2;
      const F4 mv = lds4(st + L::M2 + pt);
      const float* c = st + L::U1 + (ty + 4) * W + 4 * tx + 4;  // u^{n+1}(x0, jy, k)
      F4 out = one(c, q, r[0], mv, k);
      __syncwarp();
      if (lane == 0) mbar_arrive(&empty2[s]);  // (the stage is in registers)
      if (own) {
        const long long rel = srel0 - (long long)(k + GZ) * PS;
        if (rel >= 0 && rel < 4) {
#pragma unroll
          for (int e = 0; e < 4; ++e)
            if (rel == e) out.v[e] += a.src2.get();
        }
        st4_masked(a.uaw + (long long)(k + GZ) * PS + oc, out, x0, d.nx, true);
      }
    }
    // u^n queue: shift (plane j + 5 arrives with the next step-1 stage as r[8])
#pragma unroll
    for (int t = 0; t < 8; ++t) r[t] = r[t + 1];
  }
}

}  // namespace seis
