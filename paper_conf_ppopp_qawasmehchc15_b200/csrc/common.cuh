// common.cuh — layout, indexing and coefficients shared by the sm_100a kernels.
//
// Product path only (never includes or calls oracle/).  Paper: Qawasmeh et al.,
// PMAM'15; "P:<line>" cites /root/reference/PAPER.md, O1..O19 the readings in
// DESIGN.md §3.
//
// HBM layout.  Every state field and per-point coefficient of a
// z-slab is one fp32 array with G = 4 zero ghost cells on each side of every axis
// ("Ghost node thickness is determined by the stencil"):
//   padded dims  PX = roundup(roundup(nx, 32) + 2G, 32),  PY = roundup(ny, TY) + 2G,
//                PZ = nz_local + 2GZ,  plane stride PS = PX * PY   (G = 4, GZ = 8)
//   element (i, j, k) of the slab (interior coordinates) lives at
//                ((k + GZ) * PY + (j + G)) * PX + (i + G)
// The base pointer of each array is offset so that x = 0 of every row is
// 128-byte aligned (PX is a multiple of 32 floats).  Ghosts are never written, so
// "values outside the grid are 0" (O1) costs no branch; the 4 z-ghost planes on a
// slab face that touches a neighbour slab are the halo planes the exchange fills.
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

namespace seis {

constexpr int G = 4;     // x/y ghost width = stencil half-width (radius 4)
constexpr int GZ = 8;    // z ghost depth: 4 for the stencil + 4 for the fused acoustic kernel's
                         // recomputed q_z halo
constexpr int TXW = 32;  // tile width in x = one warp

// float count rounded up to 128 bytes (shared-memory sub-tile offsets; TMA destinations)
__host__ __device__ constexpr int r32(int n) { return (n + 31) / 32 * 32; }

struct Dims {
  int nx, ny, nzl;  // interior points of the slab
  int nz;           // global nz
  int z0;           // global z of local k = 0
  int PX, PY;       // padded pitches
  long long PS;     // plane stride
  __host__ __device__ __forceinline__ long long at(int i, int j, int k) const {
    return ((long long)(k + GZ) * PY + (j + G)) * PX + (i + G);
  }
};

// 8th-order coefficients (O1): fp32 roundings of the exact rationals
//   centred 2nd derivative c = [-205/72, 8/5, -1/5, 8/315, -1/560]
//   staggered 1st derivative d = [1225/1024, -245/3072, 49/5120, -5/7168]
// (each is a correctly rounded fp32 quotient of two exact fp32 integers).
#define SEIS_C0 (-205.0f / 72.0f)
#define SEIS_C1 (8.0f / 5.0f)
#define SEIS_C2 (-1.0f / 5.0f)
#define SEIS_C3 (8.0f / 315.0f)
#define SEIS_C4 (-1.0f / 560.0f)
#define SEIS_D1 (1225.0f / 1024.0f)
#define SEIS_D2 (-245.0f / 3072.0f)
#define SEIS_D3 (49.0f / 5120.0f)
#define SEIS_D4 (-5.0f / 7168.0f)

// Cooperative load of one plane tile of a padded field into shared memory:
// (BY + 2HY) rows x (32 + 2HX) columns starting at (i0 - HX, j0 - HY).
template <int BY, int HX, int HY>
__device__ __forceinline__ void load_tile(float* __restrict__ s, const float* __restrict__ f,
                                          long long o /* padded index of (i0, j0, k) */, int PX) {
  constexpr int W = TXW + 2 * HX;
  constexpr int H = BY + 2 * HY;
  constexpr int N = W * H;
  const int tid = threadIdx.y * TXW + threadIdx.x;
#pragma unroll
  for (int t = tid; t < N; t += TXW * BY) {
    const int r = t / W;
    const int c = t - r * W;
    s[t] = __ldg(f + o + (long long)(r - HY) * PX + (c - HX));
  }
}

// Compact C-PML memory-variable slabs (O7): psi is stored only where the
// layer can be non-zero.  W = nb + 1 points per face (the half-node layer on the
// high face is one point wider than the integer-node one).
struct CpmlIdx {
  int W;
  __device__ __forceinline__ static bool in(int i, int n, int W, bool lo) {
    return (lo && i < W) || i >= n - W;
  }
  __device__ __forceinline__ static int slot(int i, int n, int W) { return i < W ? i : i - (n - 2 * W); }
};

// Conservative, block-uniform: may the block's tile (tw x by at i0, j0) and z-chunk [k0, k1)
// hold a C-PML point (W = layer slab width per face, zlo: the top face has one)?  A block that
// may runs the full body (correct everywhere); one that does not may run the lean body.
__device__ __forceinline__ bool block_in_layers(const Dims& d, int W, int zlo, int i0, int tw, int j0, int by, int k0,
                                                int k1) {
  if (W <= 0) return false;
  const bool inner = i0 >= W && i0 + tw <= d.nx - W && j0 >= W && j0 + by <= d.ny - W &&
                     (!zlo || k0 + d.z0 >= W) && k1 + d.z0 <= d.nz - W;
  return !inner;
}

}  // namespace seis

// ----------------------------------------------------------------- TMA ring
// Plane tiles with x/y halos are brought into shared memory by the Tensor Memory
// Accelerator (cp.async.bulk.tensor.3d, completion on an mbarrier), NS stages
// deep, issued by one thread; every other operand is a coalesced register
// stream prefetched one plane ahead.
#include <cuda.h>  // CUtensorMap (type only; the driver entry point is fetched at run time)

namespace seis {

__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}
// 128-byte aligned view of a dynamic shared-memory buffer.  Pointer arithmetic
// (not an integer round trip) keeps the compiler's knowledge that the pointer is
// shared, so accesses stay LDS/STS instead of generic LD/ST.
__device__ __forceinline__ float* align128(float* p) {
  const uint32_t pad = (128u - (smem_u32(p) & 127u)) & 127u;
  return p + (pad >> 2);
}
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_fence_init() {
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t* bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes)
               : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
  asm volatile(
      "{\n"
      ".reg .pred p;\n"
      "WAIT_%=:\n"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n"
      "@!p bra WAIT_%=;\n"
      "}\n" ::"r"(smem_u32(bar)),
      "r"(parity)
      : "memory");
}
__device__ __forceinline__ void fence_proxy_async() {
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}
// Consumer release of TMA ring stage s.  With SEIS_WARP_RELEASE=1 every warp counts
// itself out of the stage once it has finished reading it, and the LAST warp re-arms the stage
// (expect_tx + TMA issue): no warp waits for the others (no CTA-wide barrier per plane).
// Default (measured faster on B200, profiles/r01_sweep4_release.jsonl): __syncthreads, then
// thread 0 re-arms.  `more` = a later plane uses stage s.
#ifndef SEIS_WARP_RELEASE
#define SEIS_WARP_RELEASE 0
#endif
#ifndef SEIS_WR_EL
#define SEIS_WR_EL SEIS_WARP_RELEASE  // the elastic kernels' choice
#endif
template <bool WR = (SEIS_WARP_RELEASE != 0), class Refill>
__device__ __forceinline__ void stage_release(uint32_t* cnt, int tid, bool more, Refill&& refill) {
  if (WR) {
  __syncwarp();
  if ((tid & 31) == 0) {
    const uint32_t nwarps = (blockDim.x * blockDim.y * blockDim.z) >> 5;
    __threadfence_block();  // this warp's reads of the stage are ordered before its count
    if (atomicAdd(cnt, 1u) == nwarps - 1) {
      atomicExch(cnt, 0u);
      __threadfence_block();
      if (more) {
        fence_proxy_async();
        refill();
      }
    }
  }
  } else {
  __syncthreads();
  if (tid == 0 && more) {
    fence_proxy_async();
    refill();
  }
  }
}
// non-blocking probe: has the phase with parity `parity` completed?
__device__ __forceinline__ bool mbar_test(uint64_t* bar, uint32_t parity) {
  uint32_t ok;
  asm volatile(
      "{\n.reg .pred p;\n"
      "mbarrier.test_wait.parity.shared::cta.b64 p, [%1], %2;\n"
      "selp.u32 %0, 1, 0, p;\n}\n"
      : "=r"(ok)
      : "r"(smem_u32(bar)), "r"(parity)
      : "memory");
  return ok != 0;
}
// producer-side wait: poll with a sleep between probes, so that a waiting producer thread does
// not take issue slots from the consumer warps of its SM sub-partition
#ifndef SEIS_AS_NAP
#define SEIS_AS_NAP 100
#endif
__device__ __forceinline__ void mbar_wait_nap(uint64_t* bar, uint32_t parity) {
  while (!mbar_test(bar, parity)) __nanosleep(SEIS_AS_NAP);
}
__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}
// 4-byte asynchronous global -> shared copy (zero-filled when !valid), and its group waits
__device__ __forceinline__ void cp_async4(float* dst, const float* src, bool valid) {
  asm volatile("cp.async.ca.shared.global [%0], [%1], 4, %2;" ::"r"(smem_u32(dst)), "l"(src), "r"(valid ? 4 : 0)
               : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
__device__ __forceinline__ void cp_async16(float* dst, const float* src) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(smem_u32(dst)), "l"(src) : "memory");
}
// wait until at most N of this thread's most recent cp.async groups are pending
template <int N>
__device__ __forceinline__ void cp_async_wait() {
  asm volatile("cp.async.wait_group %0;" ::"n"(N) : "memory");
}
// Fast reciprocal (MUFU.RCP, ~1 ulp; +inf -> +0) for the on-the-fly face/edge averages
// inter-CTA progress flags (the persistent kernels' neighbour protocol)
__device__ __forceinline__ unsigned ld_relaxed_gpu(const unsigned* p) {
  unsigned v;
  asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void fence_acq_rel_gpu() { asm volatile("fence.acq_rel.gpu;" ::: "memory"); }
__device__ __forceinline__ void prefetch_l2(const void* p) {
  asm volatile("prefetch.global.L2 [%0];" ::"l"(p));
}
__device__ __forceinline__ void red_release_gpu_add(unsigned* p, unsigned v) {
  asm volatile("red.release.gpu.global.add.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ void fence_proxy_async_global() {
  asm volatile("fence.proxy.async.global;" ::: "memory");
}

__device__ __forceinline__ float rcp_fast(float x) {
  float r;
  asm("rcp.approx.ftz.f32 %0, %1;" : "=f"(r) : "f"(x));
  return r;
}
// 3D tile load: box origin (x, y, z) in padded element coordinates
__device__ __forceinline__ void tma_load_3d(void* dst, const CUtensorMap* map, uint64_t* bar, int x, int y,
                                            int z) {
  asm volatile(
      "cp.async.bulk.tensor.3d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4, %5}], "
      "[%2];" ::"r"(smem_u32(dst)),
      "l"(reinterpret_cast<uint64_t>(map)), "r"(smem_u32(bar)), "r"(x), "r"(y), "r"(z)
      : "memory");
}

// L2 prefetch of a 3D tile (no shared-memory destination, no mbarrier): issued a few planes
// ahead of the ring so the ring's own TMA load of that plane hits in L2 (SEIS_L2PF planes).
__device__ __forceinline__ void tma_prefetch_3d(const CUtensorMap* map, int x, int y, int z) {
  asm volatile("cp.async.bulk.prefetch.tensor.3d.L2.global.tile [%0, {%1, %2, %3}];" ::"l"(
                   reinterpret_cast<uint64_t>(map)),
               "r"(x), "r"(y), "r"(z)
               : "memory");
}
__device__ __forceinline__ void tma_ld(bool pf, void* dst, const CUtensorMap* map, uint64_t* bar, int x, int y,
                                       int z) {
  if (pf) tma_prefetch_3d(map, x, y, z);
  else tma_load_3d(dst, map, bar, x, y, z);
}
#ifndef SEIS_L2PF
#define SEIS_L2PF 0
#endif
constexpr int L2PF = SEIS_L2PF;  // L2 prefetch distance beyond the TMA ring (planes), 0 = off

// Unroll factor of the z-march loops, per kernel family (u: 1 = rolled).  Unrolling by u lets
// the compiler rename the register z-queues across u planes instead of shifting them every
// plane (u-fold fewer queue moves), at u times the loop body in the instruction cache.
#define SEIS_PRAGMA_(x) _Pragma(#x)
#define SEIS_UNROLL(n) SEIS_PRAGMA_(unroll n)
#ifndef SEIS_ZU_ISO
#define SEIS_ZU_ISO 1
#endif
#ifndef SEIS_ZU_AC
#define SEIS_ZU_AC 1
#endif
#ifndef SEIS_ZU_EL
#define SEIS_ZU_EL 2  // profiles/r01_sweep_zu.jsonl: el_v -4.5 %, el_s -4.7 %; ISO / acoustic: no gain
#endif

}  // namespace seis

// ------------------------------------------------------------ 4-wide vectors
// The stencil kernels are issue-bound at one point per thread (~140 instructions
// per point); each thread therefore owns 4 consecutive x points (one float4) and
// a block tile is TXV = 64 points wide (16 threads) x BY rows.
namespace seis {

#ifndef SEIS_TXV
#define SEIS_TXV 64
#endif
constexpr int TXV = SEIS_TXV;  // ISO / acoustic tile width in x (points)
constexpr int NTX = TXV / 4;   // threads in x per block (4 points each)
constexpr int TXE = 64;        // elastic tile width in x (32 threads, 2 points each)

struct F4 {
  float v[4];
};
__device__ __forceinline__ F4 lds4(const float* p) {
  const float4 t = *reinterpret_cast<const float4*>(p);
  return F4{{t.x, t.y, t.z, t.w}};
}
__device__ __forceinline__ F4 ldg4(const float* p) {
  const float4 t = __ldg(reinterpret_cast<const float4*>(p));
  return F4{{t.x, t.y, t.z, t.w}};
}
__device__ __forceinline__ F4 ld4(const float* p) {
  const float4 t = *reinterpret_cast<const float4*>(p);
  return F4{{t.x, t.y, t.z, t.w}};
}
__device__ __forceinline__ void st4(float* p, const F4& a) {
  *reinterpret_cast<float4*>(p) = make_float4(a.v[0], a.v[1], a.v[2], a.v[3]);
}
// store the components of a group of 4 x-points that lie inside [0, nx)
__device__ __forceinline__ void st4_masked(float* p, const F4& a, int x0, int nx, bool aligned) {
  if (aligned && x0 + 3 < nx) {
    st4(p, a);
  } else {
#pragma unroll
    for (int e = 0; e < 4; ++e)
      if (x0 + e < nx) p[e] = a.v[e];
  }
}

}  // namespace seis

// 2-wide variant (the elastic kernels keep three z-queues per thread; float2 keeps
// them in registers): a block tile is TXV = 64 points wide (32 threads) x BY rows.
namespace seis {
constexpr int NTX2 = 32;
struct F2 {
  float v[2];
};
__device__ __forceinline__ F2 lds2(const float* p) {
  const float2 t = *reinterpret_cast<const float2*>(p);
  return F2{{t.x, t.y}};
}
__device__ __forceinline__ F2 ldg2(const float* p) {
  const float2 t = __ldg(reinterpret_cast<const float2*>(p));
  return F2{{t.x, t.y}};
}
__device__ __forceinline__ void st2_masked(float* p, const F2& a, int x0, int nx) {
  if (x0 + 1 < nx) {
    *reinterpret_cast<float2*>(p) = make_float2(a.v[0], a.v[1]);
  } else if (x0 < nx) {
    p[0] = a.v[0];
  }
}
}  // namespace seis

// ------------------------------------------------------ 24-bit snapshots (f2 alternative)
// Imaging reads S_j either as fp32 (s32) or in the 24-bit format of seis_shot.snap_bits = 24:
// the fp32 value rounded to nearest-even at bit 8 (sign, the full 8-bit exponent, 15 mantissa
// bits: relative rounding <= 2^-16), stored as a 16-bit high plane (h16) and an 8-bit low plane
// (l8) of the same snapshot.  The value is a pure function of the fp32 value (no scale), so
// images stay bitwise invariant under the z-slab decomposition and checkpointing.
namespace seis {
__device__ __forceinline__ uint32_t snap24_round(float v) {
  const uint32_t u = __float_as_uint(v);
  return u + 0x7Fu + ((u >> 8) & 1u);  // round to nearest even at bit 8 (then bits 0..7 drop)
}
struct SnapRef {
  const float* __restrict__ s32 = nullptr;
  const uint16_t* __restrict__ h16 = nullptr;
  const uint8_t* __restrict__ l8 = nullptr;
  __device__ __forceinline__ float at(long long i) const {
    if (h16) return __uint_as_float(((uint32_t)__ldg(h16 + i) << 16) | ((uint32_t)__ldg(l8 + i) << 8));
    return __ldg(s32 + i);
  }
};
}  // namespace seis

// ------------------------------------------------------ source amplitude (O11)
// The injected sample of step n, scale * s[n]: s is the shot's wavelet, uploaded to the device
// once per call (so a CUDA graph of the shot does not depend on the wavelet values), scale the
// per-node factor of O3 / O8 / O11.  One fp32 product, as the host would form it.
namespace seis {
struct SrcAmp {
  const float* __restrict__ w = nullptr;  // device [nt]
  int n = 0;
  float scale = 0.f;
  __device__ __forceinline__ float get() const { return __fmul_rn(scale, __ldg(w + n)); }
};
// Where a z-marching thread adds the source: the source node has padded index
// src_o (-1: none); the thread owns the `width` consecutive x points at padded column offset
// oc.  The node is the thread's point e of slab-local plane k iff
// src_o - oc - (k + GZ) PS = e in [0, width) -- at most one k since PS > width.  Resolved once
// per thread (k = -1: never) instead of a 64-bit test per plane; the same add at the same point.
struct SrcHit {
  int ke = -1;  // 4 k + e (one register), -1: never
  __device__ __forceinline__ bool at(int k) const { return (ke >> 2) == k; }
  __device__ __forceinline__ int e() const { return ke & 3; }
};
__device__ __forceinline__ SrcHit src_hit(long long src_o, long long oc, long long PS, int width) {
  SrcHit h;
  const long long r = src_o - oc;
  if (src_o >= 0 && r >= 0) {
    // m = floor(r / PS) without the 64-bit division routine: a float estimate (relative error
    // < 2^-21, so off by at most one while r / PS < 2^21 planes) and one exact correction
    long long m = (long long)((float)r * __frcp_rn((float)PS));
    long long e = r - m * PS;
    if (e < 0) {
      --m;
      e += PS;
    } else if (e >= PS) {
      ++m;
      e -= PS;
    }
    if (e < width && m >= GZ) h.ke = (int)(m - GZ) * 4 + (int)e;
  }
  return h;
}
}  // namespace seis

// ------------------------------------------------------ direct ghost-plane stores
// SURVEY §8f f4 / DESIGN.md §7: the kernel that produces an exchanged field also writes its
// first / last 4 planes straight into the neighbouring slab's ghost planes (P:175 sub-domain
// ghosts) -- another slab of this process, or another rank's slab mapped over NVLink by CUDA
// IPC -- so no separate exchange (copy, NCCL send/recv) follows the kernel.
//   lo: the slab ABOVE (smaller z); lo + (o + loo) is its bottom ghost plane nzl_lo + k for my
//       plane k < 4 (loo = nzl_lo * PS);
//   hi: the slab BELOW; hi + (o + hio) is its top ghost plane k - nzl for my plane k >= nzl - 4
//       (hio = -nzl * PS).
// nullptr = no neighbour on that side (or the ghosts travel by copies).  The padded pitches
// PX, PY are the same in every slab, so one offset per side maps a whole plane.
namespace seis {
struct Ghost {
  float* lo = nullptr;
  long long loo = 0;
  float* hi = nullptr;
  long long hio = 0;
};
#ifndef SEIS_GHOST_ST
#define SEIS_GHOST_ST 1  // 0: compile the ghost stores out (A/B timing of single-slab kernels only)
#endif
__device__ __forceinline__ void ghost_st4(const Ghost& g, long long o, int k, int nzl, const F4& v, int x0,
                                          int nx) {
  if (!SEIS_GHOST_ST) return;
  if (g.lo && k < 4) st4_masked(g.lo + (o + g.loo), v, x0, nx, true);
  if (g.hi && k >= nzl - 4) st4_masked(g.hi + (o + g.hio), v, x0, nx, true);
}
__device__ __forceinline__ void ghost_st2(const Ghost& g, long long o, int k, int nzl, const F2& v, int x0,
                                          int nx) {
  if (g.lo && k < 4) st2_masked(g.lo + (o + g.loo), v, x0, nx);
  if (g.hi && k >= nzl - 4) st2_masked(g.hi + (o + g.hio), v, x0, nx);
}
// the same for one value at padded offset o (receiver injection): the ghost copy receives the
// value the owner stored, so both sides hold bitwise the same number
__device__ __forceinline__ void ghost_st1(const Ghost& g, long long o, int k, int nzl, float v) {
  if (g.lo && k < 4) g.lo[o + g.loo] = v;
  if (g.hi && k >= nzl - 4) g.hi[o + g.hio] = v;
}
}  // namespace seis

// ------------------------------------------------ C-PML memory-variable access
// psi values are first-touch global data inside the layers; the kernels load the old
// values BEFORE waiting for the plane's TMA stage (so their latency overlaps the wait
// and the derivative arithmetic) and store the updated values afterwards.
namespace seis {

// compact-slab indices of the NV points of a group (or -1 outside the layer / grid).
// 32-bit: a compact slab holds < 2^31 points up to 1024^3 grids (checked at create).
template <int NV>
__device__ __forceinline__ void psi_idx_x(int* ix, const Dims& d, int W, int x0, int j, int k) {
#pragma unroll
  for (int e = 0; e < NV; ++e) {
    const int x = x0 + e;
    ix[e] = (x < d.nx && CpmlIdx::in(x, d.nx, W, true)) ? (k * d.ny + j) * (2 * W) + CpmlIdx::slot(x, d.nx, W)
                                                          : -1;
  }
}
template <int NV>
__device__ __forceinline__ void psi_idx_row(int* ix, int base, int x0, int nx) {
#pragma unroll
  for (int e = 0; e < NV; ++e) ix[e] = (x0 + e < nx) ? base + e : -1;
}
template <int NV>
__device__ __forceinline__ void psi_ld(float* old, const float* __restrict__ ps, const int* ix) {
#pragma unroll
  for (int e = 0; e < NV; ++e) old[e] = ix[e] >= 0 ? ps[ix[e]] : 0.0f;
}
// The x / y C-PML coefficients (a, b, ah, bh) of a block's TW columns and BY rows, staged in
// shared memory once per block: the z-march uses them on every plane, and a shared load has
// a short fixed latency where the global (L1) load it replaces sat on the critical path
// after the stage wait.
template <int TW, int BY>
struct CpmlTile {
  float x[4][TW];
  float y[4][BY];
};
template <int TW, int BY, class Axis>
__device__ __forceinline__ void cpml_tile_fill(CpmlTile<TW, BY>& t, const Axis& cx, const Axis& cy, int i0,
                                               int j0, int nx, int ny, bool on, int tid, int nthr) {
  if (!on) return;
  for (int q = tid; q < 4 * TW; q += nthr) {
    const int r = q / TW, c = q - r * TW;
    const int x = min(i0 + c, nx - 1);
    const float* p = r == 0 ? cx.a : (r == 1 ? cx.b : (r == 2 ? cx.ah : cx.bh));
    t.x[r][c] = __ldg(p + x);
  }
  for (int q = tid; q < 4 * BY; q += nthr) {
    const int r = q / BY, c = q - r * BY;
    const int y = min(j0 + c, ny - 1);
    const float* p = r == 0 ? cy.a : (r == 1 ? cy.b : (r == 2 ? cy.ah : cy.bh));
    t.y[r][c] = __ldg(p + y);
  }
}

// psi <- b psi + a dv;  dv += psi   (per point coefficients ca[e], cb[e])
template <int NV>
__device__ __forceinline__ void psi_upd(float* dv, float* __restrict__ ps, const int* ix, const float* old,
                                        const float* ca, const float* cb) {
#pragma unroll
  for (int e = 0; e < NV; ++e)
    if (ix[e] >= 0) {
      const float v = fmaf(cb[e], old[e], ca[e] * dv[e]);
      ps[ix[e]] = v;
      dv[e] += v;
    }
}
// y / z slab rows: the group's NV values are contiguous (ix[e] = ix[0] + e); with the whole
// group inside the grid and NV-aligned rows (vec: x0 + NV - 1 < nx, nx % NV == 0) one NV-wide
// load / store instead of NV scalar ones (the same values, the same arithmetic)
template <int NV>
__device__ __forceinline__ void psi_ld_row(float* old, const float* __restrict__ ps, const int* ix, bool vec) {
  static_assert(NV == 2 || NV == 4, "2- or 4-wide groups");
  if (vec) {
    if constexpr (NV == 4) {
      const float4 t = *reinterpret_cast<const float4*>(ps + ix[0]);
      old[0] = t.x;
      old[1] = t.y;
      old[2] = t.z;
      old[3] = t.w;
    } else {
      const float2 t = *reinterpret_cast<const float2*>(ps + ix[0]);
      old[0] = t.x;
      old[1] = t.y;
    }
  } else {
    psi_ld<NV>(old, ps, ix);
  }
}
template <int NV>
__device__ __forceinline__ void psi_upd_row(float* dv, float* __restrict__ ps, const int* ix, const float* old,
                                            const float* ca, const float* cb, bool vec) {
  if (vec) {
    float v[NV];
#pragma unroll
    for (int e = 0; e < NV; ++e) {
      v[e] = fmaf(cb[e], old[e], ca[e] * dv[e]);
      dv[e] += v[e];
    }
    if constexpr (NV == 4) *reinterpret_cast<float4*>(ps + ix[0]) = make_float4(v[0], v[1], v[2], v[3]);
    else *reinterpret_cast<float2*>(ps + ix[0]) = make_float2(v[0], v[1]);
  } else {
    psi_upd<NV>(dv, ps, ix, old, ca, cb);
  }
}

}  // namespace seis
