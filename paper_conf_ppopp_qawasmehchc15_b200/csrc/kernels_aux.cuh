// kernels_aux.cuh — receiver sampling, receiver injection (P:206,
// P:330) and small helpers.
//
// Receiver injection is ONE launch per step over all receivers (the paper's
// per-receiver launches took 26.2% of GPU time; its suggested fix).
// Duplicate receiver positions are merged on the host into groups (CSR): each
// distinct node is updated by exactly one thread, summing its receivers'
// samples in receiver-index order (O12), so there are no atomics and no races.
#pragma once
#include "common.cuh"

namespace seis {

// seis_row[r] = f[off[r]] for the receivers this slab owns (off[r] >= 0).
// Elastic pressure (component 3): -(f0 + f1 + f2)/3 at the node.
__global__ void gather_kernel(float* __restrict__ seis_row, const float* __restrict__ f0,
                              const float* __restrict__ f1, const float* __restrict__ f2,
                              const long long* __restrict__ off, const int* __restrict__ rid, int n,
                              int pressure) {
  const int t = blockIdx.x * blockDim.x + threadIdx.x;
  if (t >= n) return;
  const long long o = off[t];
  float v;
  if (pressure) {
    v = -(f0[o] + f1[o] + f2[o]) / 3.0f;
  } else {
    v = f0[o];
  }
  seis_row[rid[t]] = v;
}

// Backward-phase receiver injection (O15), ISO and ACOUSTIC: for each distinct node u of this
// slab, f[off[u]] += scale[u] * sum_{r in group u, index order} data_row[r]
// (ELASTIC receivers inject like the explosive source: inject_el_kernel below.)
__global__ void inject_kernel(float* __restrict__ f, const long long* __restrict__ off,
                              const float* __restrict__ scale, const int* __restrict__ gstart,
                              const int* __restrict__ members, const float* __restrict__ data_row,
                              int ngroups, Ghost gh, long long PS, int nzl,
                              const int* __restrict__ sidx, float* __restrict__ spx) {
  const int u = blockIdx.x * blockDim.x + threadIdx.x;
  if (u >= ngroups) return;
  float s = 0.0f;
  for (int t = gstart[u]; t < gstart[u + 1]; ++t) s += data_row[members[t]];
  const long long o = off[u];
  const float v = fmaf(scale[u], s, f[o]);
  f[o] = v;
  if (spx && sidx[u] >= 0) spx[sidx[u]] = fmaf(scale[u], s, spx[sidx[u]]);  // ISO O6b: x component
  ghost_st1(gh, o, (int)(o / PS) - GZ, nzl, v);  // (f4) the neighbour's ghost copy of the node
}

// Elastic RTM receiver injection (f3): receivers act like the explosive source (O11),
//   s_ii -= scale[u] * sum_{r in group u} data_row[r]   for ii = xx, yy, zz,
// except s_zz on a free-surface node, which the surface condition keeps at 0 (O16).
__global__ void inject_el_kernel(float* __restrict__ sxx, float* __restrict__ syy, float* __restrict__ szz,
                                 const long long* __restrict__ off, const float* __restrict__ scale,
                                 const int* __restrict__ gstart, const int* __restrict__ members,
                                 const float* __restrict__ data_row, const int* __restrict__ surf,
                                 int ngroups, Ghost gh, long long PS, int nzl) {
  const int u = blockIdx.x * blockDim.x + threadIdx.x;
  if (u >= ngroups) return;
  float s = 0.0f;
  for (int t = gstart[u]; t < gstart[u + 1]; ++t) s += data_row[members[t]];
  const long long o = off[u];
  const float v = scale[u] * s;
  sxx[o] -= v;
  syy[o] -= v;
  if (!surf[u]) {
    const float z = szz[o] - v;
    szz[o] = z;
    ghost_st1(gh, o, (int)(o / PS) - GZ, nzl, z);  // (f4) only szz of the three is exchanged
  }
}

// 24-bit snapshots (SURVEY §8f f2's compressed-snapshot alternative, seis_shot.snap_bits = 24):
// the snapshot field S = f0 (ISO / ACOUSTIC) or the pressure -(sxx+syy+szz)/3 (ELASTIC, the
// el_s SNAP epilogue's expression) rounded to 24 bits (common.cuh snap24_round) and split into
// the high 16 bits (hi) and the next 8 bits (lo) of the fp32 pattern: 3 bytes per value.
__device__ __forceinline__ float snap_val(const float* f0, const float* f1, const float* f2, int nf, long long o) {
  return nf == 1 ? f0[o] : -((f0[o] + f1[o]) + f2[o]) / 3.0f;
}
__global__ void snap24_kernel(uint16_t* __restrict__ hi, uint8_t* __restrict__ lo, const float* __restrict__ f0,
                              const float* __restrict__ f1, const float* __restrict__ f2, int nf, Dims d) {
  const long long n = (long long)d.nzl * d.ny * d.nx;
  for (long long t = blockIdx.x * (long long)blockDim.x + threadIdx.x; t < n; t += (long long)gridDim.x * blockDim.x) {
    const int i = (int)(t % d.nx);
    const long long r = t / d.nx;
    const uint32_t u = snap24_round(snap_val(f0, f1, f2, nf, d.at(i, (int)(r % d.ny), (int)(r / d.ny))));
    hi[t] = (uint16_t)(u >> 16);
    lo[t] = (uint8_t)(u >> 8);
  }
}

// Copy the interior of a padded slab field to a compact [nzl][ny][nx] array.
__global__ void unpad_kernel(float* __restrict__ dst, const float* __restrict__ src, Dims d) {
  const long long n = (long long)d.nzl * d.ny * d.nx;
  for (long long t = blockIdx.x * (long long)blockDim.x + threadIdx.x; t < n;
       t += (long long)gridDim.x * blockDim.x) {
    const int i = (int)(t % d.nx);
    const long long r = t / d.nx;
    const int j = (int)(r % d.ny);
    const int k = (int)(r / d.ny);
    dst[t] = src[d.at(i, j, k)];
  }
}

// Scatter a compact [nzl][ny][nx] fp32 array into the interior of a padded array.
__global__ void pad_kernel(float* __restrict__ dst, const float* __restrict__ src, Dims d) {
  const long long n = (long long)d.nzl * d.ny * d.nx;
  for (long long t = blockIdx.x * (long long)blockDim.x + threadIdx.x; t < n;
       t += (long long)gridDim.x * blockDim.x) {
    const int i = (int)(t % d.nx);
    const long long r = t / d.nx;
    const int j = (int)(r % d.ny);
    const int k = (int)(r / d.ny);
    dst[d.at(i, j, k)] = src[t];
  }
}

}  // namespace seis
