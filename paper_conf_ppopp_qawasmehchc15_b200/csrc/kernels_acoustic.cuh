// kernels_acoustic.cuh — Eq 2 in 3D: variable-density acoustic,
// first-order staggered system, leapfrog (O2, O8), C-PML (O7).
//
//   V:  psi_{p,d} <- bh_d psi_{p,d} + ah_d D+_d p;   q_d += (dt b_d / h)(D+_d p + psi_{p,d})
//   P:  psi_{q,d} <- b_d  psi_{q,d} + a_d  D-_d q_d;  p += (dt K / h) sum_d (D-_d q_d + psi_{q,d})
// with h D+ f_{i+1/2} = sum_m d_m (f_{i+m} - f_{i-m+1}), h D- g_i = sum_m d_m (g_{i+m-1} - g_{i-m})
// (psi is stored multiplied by h, so both updates work on the unscaled differences).
//
// One fused z-marching kernel per time step (ac_step_kernel, below).
// Fused epilogues: the source, the snapshot store and the
// imaging condition on the input p (O15).
#pragma once
#include "common.cuh"

namespace seis {

struct CpmlAxis {
  const float* __restrict__ a;   // integer nodes
  const float* __restrict__ b;
  const float* __restrict__ ah;  // half nodes i + 1/2
  const float* __restrict__ bh;
};

// ---------------------------------------------------------------------------
// Fused single-sweep acoustic step: one z-march computes
// q^{n+1/2} = V(p^n, q^{n-1/2}) and p^{n+1} = P(p^n, q^{n+1/2}) in the same pass.
// The x/y halos of q^{n+1/2} that P needs (4 points per side, x for q_x, y for
// q_y) are recomputed from the p^n tile (halo 8) instead of being read back, and
// q_z^{n+1/2} comes out of the z-march 3 planes ahead of the P update (register
// queue).  State is double-buffered (A = step input, B = output) so recomputed
// halo values always see the step's inputs; C-PML psi_p (read at recomputed
// points) is double-buffered too, psi_q is only touched by its owner (in place).
// Per point HBM traffic: read p^n, q^{n-1/2} x3, rho, dt K/h; write p^{n+1},
// q^{n+1/2} x3 = 40 B (vs 56 B for the two-kernel V + P form with rho).
// Buoyancy dt b/h = (dt/h) 2/(rho_i + rho_{i+1}) is evaluated on the fly (O8).
// Bitwise identical to itself under any tiling / z-chunking / slab split: a
// recomputed halo value is the same expression on the same inputs as the owner's.
struct AcFArgs {
  CUtensorMap mp;                  // p^n tile, box (32+16) x (BY+16): x from i0-8, y from j0-8
  CUtensorMap mr;                  // rho tile, same box
  CUtensorMap mqx;                 // q_x^{n-1/2}, box (32+8) x BY: x from i0-4
  CUtensorMap mqy;                 // q_y^{n-1/2}, box 32 x (BY+8): y from j0-4
  CUtensorMap mk;                  // dt K / h, box 32 x BY
  const float* __restrict__ pA;    // p^n (padded)
  const float* __restrict__ qzA;   // q_z^{n-1/2}
  const float* __restrict__ rho;   // density (padded, z ghosts filled from neighbours)
  float* __restrict__ pB;
  float* __restrict__ qxB;
  float* __restrict__ qyB;
  float* __restrict__ qzB;
  float dth;                       // dt / h
  int W, zlo;
  CpmlAxis cx, cy, cz;
  const float* __restrict__ psxA;  // psi_{p,x} [nzl][ny][2W] (input)
  const float* __restrict__ psyA;  // psi_{p,y} [nzl][2W][nx]
  const float* __restrict__ pszA;  // psi_{p,z} [2W][ny][nx]
  float* __restrict__ psxB;
  float* __restrict__ psyB;
  float* __restrict__ pszB;
  float* __restrict__ pqx;         // psi_{q,*}, owner-only (in place)
  float* __restrict__ pqy;
  float* __restrict__ pqz;
  Dims d;
  int zc;
  long long src_o;
  float src_amp;
  float* __restrict__ snap;
  const float* __restrict__ imgS;
  float* __restrict__ img;
};

constexpr int ACF_NS = 3;

template <int BY>
struct AcFStage {
  static constexpr int PW = TXW + 16, PH = BY + 16, QXW = TXW + 8, QYH = BY + 8, T = TXW * BY;
  static constexpr int P = 0, R = PW * PH, QX = 2 * PW * PH, QY = QX + QXW * BY, K = QY + TXW * QYH,
                       SIZE = K + T;
  static constexpr int SCRATCH = QXW * BY + TXW * QYH;  // q_x, q_y at step n+1/2 incl. halos
  static constexpr size_t smem_bytes() { return ((size_t)ACF_NS * SIZE + SCRATCH) * 4 + 128; }
};

// buoyancy on a face: (dt/h) * 2 / (rho0 + rho1)
__device__ __forceinline__ float face_b(float dth, float r0, float r1) { return dth * (2.0f / (r0 + r1)); }

template <int BY, bool SNAP, bool IMG>
__global__ void __launch_bounds__(TXW * BY) ac_step_kernel(const __grid_constant__ AcFArgs a) {
  using L = AcFStage<BY>;
  constexpr int PW = L::PW, QXW = L::QXW;
  constexpr uint32_t TX_BYTES = L::SIZE * 4;
  constexpr int NT = TXW * BY;
  extern __shared__ __align__(128) float sm_raw[];
  float* sm = align128(sm_raw);
  float* qxn = sm + ACF_NS * L::SIZE;   // [BY][QXW]   q_x^{n+1/2}, x from i0-4
  float* qyn = qxn + QXW * BY;          // [BY+8][TXW] q_y^{n+1/2}, y from j0-4
  __shared__ __align__(8) uint64_t bar[ACF_NS];
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
  const int Wl = a.W;
  const float dth = a.dth;
  auto issue = [&](int s, int k) {
    float* st = sm + s * L::SIZE;
    const int z = k + GZ;
    mbar_expect_tx(&bar[s], TX_BYTES);
    tma_load_3d(st + L::P, &a.mp, &bar[s], i0 - 4, j0 - 4, z);
    tma_load_3d(st + L::R, &a.mr, &bar[s], i0 - 4, j0 - 4, z);
    tma_load_3d(st + L::QX, &a.mqx, &bar[s], i0, j0 + G, z);
    tma_load_3d(st + L::QY, &a.mqy, &bar[s], i0 + G, j0, z);
    tma_load_3d(st + L::K, &a.mk, &bar[s], i0 + G, j0 + G, z);
  };
  if (tid == 0) {
    for (int s = 0; s < ACF_NS; ++s) mbar_init(&bar[s], 1);
    mbar_fence_init();
  }
  __syncthreads();
  if (tid == 0)
    for (int s = 0; s < ACF_NS && s < np; ++s) issue(s, k0 + s);

  const float* __restrict__ pA = a.pA;
  const float* __restrict__ qzA = a.qzA;
  const float* __restrict__ rho = a.rho;
  // q_z^{n+1/2} at plane kk from p^n(kk-3 .. kk+4) = w[0..7], rho(kk), rho(kk+1), q_z^{n-1/2}(kk)
  auto qz_new = [&](int kk, const float* w, float r0, float r1, float qold) -> float {
    const int gz = kk + d.z0;
    if (!own || gz < 0 || gz >= d.nz) return 0.0f;
    float dz = SEIS_D1 * (w[4] - w[3]);
    dz = fmaf(SEIS_D2, w[5] - w[2], dz);
    dz = fmaf(SEIS_D3, w[6] - w[1], dz);
    dz = fmaf(SEIS_D4, w[7] - w[0], dz);
    if (Wl > 0 && CpmlIdx::in(gz, d.nz, Wl, a.zlo)) {
      const long long iz = ((long long)CpmlIdx::slot(gz, d.nz, Wl) * d.ny + j) * d.nx + i;
      const float ps = fmaf(__ldg(a.cz.bh + gz), a.pszA[iz], __ldg(a.cz.ah + gz) * dz);
      if (kk >= k0 && kk < k1) a.pszB[iz] = ps;
      dz += ps;
    }
    const float b = face_b(dth, r0, gz + 1 < d.nz ? r1 : r0);
    const float v = fmaf(b, dz, qold);
    if (kk >= k0 && kk < k1) a.qzB[(long long)(kk + GZ) * PS + oc] = v;
    return v;
  };

  // warm-up: q_z^{n+1/2} at planes k0-4 .. k0+2 (needs p^n at k0-7 .. k0+6)
  float pq[8];   // p^n(k .. k+7) at the start of iteration k
  float qzq[8];  // q_z^{n+1/2}(k-4 .. k+3)
  float rq0;     // rho(k+3)
  {
    float w[14];
#pragma unroll
    for (int t = 0; t < 14; ++t) w[t] = __ldg(pA + (long long)(k0 - 7 + t + GZ) * PS + oc);
    float rr[8];
#pragma unroll
    for (int t = 0; t < 8; ++t) rr[t] = __ldg(rho + (long long)(k0 - 4 + t + GZ) * PS + oc);
#pragma unroll
    for (int t = 0; t < 7; ++t) {
      const float qo = __ldg(qzA + (long long)(k0 - 4 + t + GZ) * PS + oc);
      qzq[t] = qz_new(k0 - 4 + t, w + t, rr[t], rr[t + 1], qo);
    }
#pragma unroll
    for (int t = 0; t < 7; ++t) pq[t] = w[7 + t];
    rq0 = rr[7];  // rho(k0+3)
  }
  pq[7] = __ldg(pA + (long long)(k0 + 7 + GZ) * PS + oc);
  float rq1 = __ldg(rho + (long long)(k0 + 4 + GZ) * PS + oc);
  float qzo = __ldg(qzA + (long long)(k0 + 3 + GZ) * PS + oc);
  const bool lxo = Wl > 0 && CpmlIdx::in(i, d.nx, Wl, true);
  const bool lyo = Wl > 0 && CpmlIdx::in(j, d.ny, Wl, true);

  for (int it = 0; it < np; ++it) {
    const int k = k0 + it;
    const int s = it % ACF_NS;
    const long long o = (long long)(k + GZ) * PS + oc;
    // next plane's streams (one ahead)
    float p_next = 0.f, r_next = 0.f, qz_next = 0.f;
    if (it + 1 < np) {
      p_next = __ldg(pA + o + 8 * PS);
      r_next = __ldg(rho + o + 5 * PS);
      qz_next = __ldg(qzA + o + 4 * PS);
    }
    mbar_wait(&bar[s], (it / ACF_NS) & 1);
    const float* st = sm + s * L::SIZE;
    // ---- V: q_x^{n+1/2} on the tile plus its x halo (x from i0-4, QXW wide) ----
    for (int t = tid; t < QXW * BY; t += NT) {
      const int r = t / QXW, c = t - r * QXW;
      const int x = i0 - 4 + c, y = j0 + r;
      const float* pc = st + L::P + (r + 8) * PW + (c + 4);
      float dx = SEIS_D1 * (pc[1] - pc[0]);
      dx = fmaf(SEIS_D2, pc[2] - pc[-1], dx);
      dx = fmaf(SEIS_D3, pc[3] - pc[-2], dx);
      dx = fmaf(SEIS_D4, pc[4] - pc[-3], dx);
      float v = 0.0f;
      if (x >= 0 && x < d.nx && y < d.ny) {
        const bool ownpt = c >= 4 && c < 4 + TXW;
        if (Wl > 0 && CpmlIdx::in(x, d.nx, Wl, true)) {
          const long long ix = ((long long)k * d.ny + y) * (2 * Wl) + CpmlIdx::slot(x, d.nx, Wl);
          const float ps = fmaf(__ldg(a.cx.bh + x), a.psxA[ix], __ldg(a.cx.ah + x) * dx);
          if (ownpt) a.psxB[ix] = ps;
          dx += ps;
        }
        const float* rc = st + L::R + (r + 8) * PW + (c + 4);
        const float b = face_b(dth, rc[0], x + 1 < d.nx ? rc[1] : rc[0]);
        v = fmaf(b, dx, st[L::QX + t]);
        if (ownpt) a.qxB[(long long)(k + GZ) * PS + (long long)(y + G) * d.PX + (x + G)] = v;
      }
      qxn[t] = v;
    }
    // ---- V: q_y^{n+1/2} on the tile plus its y halo (y from j0-4) ----
    for (int t = tid; t < TXW * (BY + 8); t += NT) {
      const int r = t / TXW, c = t - r * TXW;
      const int x = i0 + c, y = j0 - 4 + r;
      const float* pc = st + L::P + (r + 4) * PW + (c + 8);
      float dy = SEIS_D1 * (pc[PW] - pc[0]);
      dy = fmaf(SEIS_D2, pc[2 * PW] - pc[-PW], dy);
      dy = fmaf(SEIS_D3, pc[3 * PW] - pc[-2 * PW], dy);
      dy = fmaf(SEIS_D4, pc[4 * PW] - pc[-3 * PW], dy);
      float v = 0.0f;
      if (y >= 0 && y < d.ny && x < d.nx) {
        const bool ownpt = r >= 4 && r < 4 + BY;
        if (Wl > 0 && CpmlIdx::in(y, d.ny, Wl, true)) {
          const long long iy = ((long long)k * (2 * Wl) + CpmlIdx::slot(y, d.ny, Wl)) * d.nx + x;
          const float ps = fmaf(__ldg(a.cy.bh + y), a.psyA[iy], __ldg(a.cy.ah + y) * dy);
          if (ownpt) a.psyB[iy] = ps;
          dy += ps;
        }
        const float* rc = st + L::R + (r + 4) * PW + (c + 8);
        const float b = face_b(dth, rc[0], y + 1 < d.ny ? rc[PW] : rc[0]);
        v = fmaf(b, dy, st[L::QY + t]);
        if (ownpt) a.qyB[(long long)(k + GZ) * PS + (long long)(y + G) * d.PX + (x + G)] = v;
      }
      qyn[t] = v;
    }
    // ---- V: q_z^{n+1/2} at plane k+3 (z-march, register queue) ----
    qzq[7] = qz_new(k + 3, pq, rq0, rq1, qzo);
    __syncthreads();
    // ---- P: p^{n+1} at plane k ----
    if (own) {
      const float* cx = qxn + ty * QXW + tx + 4;
      const float* cy = qyn + (ty + 4) * TXW + tx;
      float dx = SEIS_D1 * (cx[0] - cx[-1]);
      dx = fmaf(SEIS_D2, cx[1] - cx[-2], dx);
      dx = fmaf(SEIS_D3, cx[2] - cx[-3], dx);
      dx = fmaf(SEIS_D4, cx[3] - cx[-4], dx);
      float dy = SEIS_D1 * (cy[0] - cy[-TXW]);
      dy = fmaf(SEIS_D2, cy[TXW] - cy[-2 * TXW], dy);
      dy = fmaf(SEIS_D3, cy[2 * TXW] - cy[-3 * TXW], dy);
      dy = fmaf(SEIS_D4, cy[3 * TXW] - cy[-4 * TXW], dy);
      float dz = SEIS_D1 * (qzq[4] - qzq[3]);
      dz = fmaf(SEIS_D2, qzq[5] - qzq[2], dz);
      dz = fmaf(SEIS_D3, qzq[6] - qzq[1], dz);
      dz = fmaf(SEIS_D4, qzq[7] - qzq[0], dz);
      if (Wl > 0) {
        if (lxo) {
          const long long ix = ((long long)k * d.ny + j) * (2 * Wl) + CpmlIdx::slot(i, d.nx, Wl);
          const float ps = fmaf(__ldg(a.cx.b + i), a.pqx[ix], __ldg(a.cx.a + i) * dx);
          a.pqx[ix] = ps;
          dx += ps;
        }
        if (lyo) {
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
      float out = fmaf(st[L::K + tid], (dx + dy) + dz, pq[0]);
      if (o == a.src_o) out += a.src_amp;
      a.pB[o] = out;
      if (SNAP || IMG) {
        const long long cix = ((long long)k * d.ny + j) * d.nx + i;
        if (SNAP) a.snap[cix] = out;
        if (IMG) a.img[cix] = fmaf(__ldg(a.imgS + cix), pq[0], a.img[cix]);
      }
    }
    __syncthreads();  // stage s and the q scratch are free
    if (tid == 0 && it + ACF_NS < np) {
      fence_proxy_async();
      issue(s, k + ACF_NS);
    }
#pragma unroll
    for (int t = 0; t < 7; ++t) {
      pq[t] = pq[t + 1];
      qzq[t] = qzq[t + 1];
    }
    pq[7] = p_next;
    rq0 = rq1;
    rq1 = r_next;
    qzo = qz_next;
  }
}

}  // namespace seis
