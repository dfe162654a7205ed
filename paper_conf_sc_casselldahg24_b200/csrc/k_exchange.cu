// k_exchange.cu -- K7 fused with the multi-GPU exchange.
//
// Alg. 6 ends every step with the leapfrog update; on G ranks
// each rank updates only its Hilbert range [A21] and the next step needs the
// full state on every rank.  Instead of a leapfrog kernel followed by an
// all-gather, the update kernel stores each new record directly into the
// same slot of every rank's state buffer (peer memory over NVLink/NVSwitch),
// so the exchange overlaps the arithmetic store by store.  Two device-side
// barriers per step order it against the readers:
//   slot 0  after the permute: every rank has consumed its copy of the old
//           state, so peers may overwrite it;
//   slot 1  after the update: every rank's stores have landed.
#include <cuda_runtime.h>

#include <cstdint>

#include "internal.cuh"

namespace nb {
namespace {

__device__ __forceinline__ void st_release_sys(unsigned* p, unsigned v) {
  asm volatile("st.release.sys.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}

__device__ __forceinline__ unsigned ld_acquire_sys(const unsigned* p) {
  unsigned v;
  asm volatile("ld.acquire.sys.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}

__device__ __forceinline__ uint64_t global_ns() {
  uint64_t t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}

__global__ __launch_bounds__(256) void k_leapfrog_scatter(const float4* __restrict__ pm_in,
                                                          const float4* __restrict__ vi_in,
                                                          const float4* __restrict__ acc, int64_t b, int64_t len,
                                                          float dt, PeerTable pt, const int64_t* __restrict__ part) {
  if (part) {  // NEXT-3(i): this step's range, decided on the device
    b = part[pt.rank];
    len = part[pt.rank + 1] - b;
  }
  const int64_t i = int64_t(blockIdx.x) * blockDim.x + threadIdx.x;
  if (i >= len) return;
  float4 p = pm_in[b + i], v = vi_in[b + i];
  const float4 a = acc[i];
  // same operations, same order as k_leapfrog (results bit-identical to G = 1)
  v.x = fmaf(a.x, dt, v.x);
  v.y = fmaf(a.y, dt, v.y);
  v.z = fmaf(a.z, dt, v.z);
  p.x = fmaf(v.x, dt, p.x);
  p.y = fmaf(v.y, dt, p.y);
  p.z = fmaf(v.z, dt, p.z);
#pragma unroll
  for (int r = 0; r < kMaxPeers; ++r) {
    if (r < pt.G) {
      pt.pm[r][b + i] = p;
      pt.vi[r][b + i] = v;
    }
  }
}

// NEXT-3(i) cost-weighted Hilbert ranges.  Unit u (256
// slots = 8 warp groups of 32, the partition unit of [A21]) costs w_u = the
// interaction count of its slots in the last pass (the sum of its groups'
// costs; identical data on every rank after the delivery barrier).  With
// E_u = sum_{i<u} w_i and W = E_U, boundary r is B_r = min{ u : E_u >=
// ceil(r W / G) }, then clamped in rank order so that every slice has at
// most cap units and the remaining ranks can still cover the rest; slot
// boundary = min(n, 256 B_r).  One block: each thread sums a contiguous
// chunk of units, a block scan of the chunk sums locates the chunk holding
// each target, whose thread walks it.
constexpr int kPartThreads = 1024;
constexpr int kUnitGroups = kPartUnitSlots / 32;  // 32-slot cost groups per partition unit

__device__ __forceinline__ unsigned long long unit_cost(const uint32_t* __restrict__ w, int64_t J, int64_t u) {
  unsigned long long c = 0;
  const int64_t j1 = min(J, (u + 1) * kUnitGroups);
  for (int64_t j = u * kUnitGroups; j < j1; ++j) c += w[j];
  return c;
}

__global__ __launch_bounds__(kPartThreads) void k_partition(const uint32_t* __restrict__ w, int64_t J, int G,
                                                            int64_t n, int64_t cap, int64_t* __restrict__ part,
                                                            int64_t* __restrict__ used) {
  __shared__ unsigned long long s_pre[kPartThreads + 1];
  __shared__ int64_t s_B[kMaxPeers + 1];
  const int t = threadIdx.x;
  const int64_t U = (J + kUnitGroups - 1) / kUnitGroups;
  const int64_t chunk = (U + kPartThreads - 1) / kPartThreads;
  const int64_t u0 = min(U, int64_t(t) * chunk), u1 = min(U, u0 + chunk);
  unsigned long long sum = 0;
  for (int64_t u = u0; u < u1; ++u) sum += unit_cost(w, J, u);
  s_pre[t + 1] = sum;
  if (t == 0) s_pre[0] = 0;
  __syncthreads();
  for (int o = 1; o < kPartThreads; o <<= 1) {  // inclusive scan of s_pre[1..]
    const unsigned long long v = t >= o ? s_pre[t + 1 - o] : 0ull;
    __syncthreads();
    s_pre[t + 1] += v;
    __syncthreads();
  }
  const unsigned long long W = s_pre[kPartThreads];
  // thread t owns targets with s_pre[t] < target <= s_pre[t + 1]
  for (int r = 1; r < G; ++r) {
    using u64 = unsigned long long;
    const u64 target = (W * u64(r) + u64(G) - 1) / u64(G);
    if (target == 0) {
      if (t == 0) s_B[r] = 0;
    } else if (s_pre[t] < target && target <= s_pre[t + 1]) {
      unsigned long long e = s_pre[t];
      int64_t u = u0;
      while (e < target) e += unit_cost(w, J, u++);  // E_u >= target first at this u
      s_B[r] = u;
    }
  }
  __syncthreads();
  if (t == 0) {
    s_B[0] = 0;
    s_B[G] = U;
    for (int r = 1; r < G; ++r) {
      int64_t b = s_B[r];
      b = max(b, s_B[r - 1]);
      b = min(b, s_B[r - 1] + cap);
      b = max(b, U - int64_t(G - r) * cap);
      s_B[r] = b;
    }
    for (int r = 0; r <= G; ++r) {
      used[r] = part[r];
      part[r] = min(n, int64_t(kUnitGroups) * 32 * s_B[r]);
    }
  }
}

__global__ void k_xbarrier(PeerTable pt, unsigned* epoch, int slot, int* err) {
  __shared__ unsigned ep;
  if (threadIdx.x == 0) {
    ep = epoch[slot] + 1;
    epoch[slot] = ep;
  }
  __syncthreads();
  const int q = threadIdx.x;
  if (q >= pt.G) return;
  // release: this rank's earlier stores (the previous kernels in stream
  // order, peer stores included) are visible before the signal
  __threadfence_system();
  st_release_sys(pt.flags[q] + slot * kMaxPeers + pt.rank, ep);
  const unsigned* f = pt.flags[pt.rank] + slot * kMaxPeers + q;
  if (*reinterpret_cast<volatile int*>(err)) return;  // a peer already timed out: do not hang again
  const uint64_t t0 = global_ns();
  while (int(ld_acquire_sys(f) - ep) < 0) {  // epochs only grow (wrap-safe compare)
    __nanosleep(200);
    if (global_ns() - t0 > 20ull * 1000000000ull) {
      atomicExch(err, 1);
      return;
    }
  }
}

}  // namespace

void launch_leapfrog_scatter(const float4* pm_in, const float4* vi_in, const float4* acc, int64_t b, int64_t len,
                             float dt, const PeerTable& pt, const int64_t* part, cudaStream_t s) {
  if (len <= 0) return;
  k_leapfrog_scatter<<<unsigned((len + 255) / 256), 256, 0, s>>>(pm_in, vi_in, acc, b, len, dt, pt, part);
}

void launch_partition(const uint32_t* gcost, int64_t groups, int G, int64_t n, int64_t cap_units, int64_t* part,
                      int64_t* used, cudaStream_t s) {
  k_partition<<<1, kPartThreads, 0, s>>>(gcost, groups, G, n, cap_units, part, used);
}

void launch_xbarrier(const PeerTable& pt, unsigned* epoch, int slot, int* err, cudaStream_t s) {
  k_xbarrier<<<1, 32, 0, s>>>(pt, epoch, slot, err);
}


// Load every kernel of this file now (see preload_all in capi.cu).
void preload_exchange() {
  touch(k_leapfrog_scatter);
  touch(k_partition);
  touch(k_xbarrier);
}

}  // namespace nb
