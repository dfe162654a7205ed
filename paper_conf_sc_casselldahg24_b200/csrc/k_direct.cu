// NEXT-1: the paper's All-Pairs baseline (direct
// summation of Eq. 1) as a GPU kernel, for sampled targets, with fp64
// arithmetic and accumulation -- the exact reference the theta sweep measures
// Barnes-Hut accuracy against (config 5).  Tiled over sources in shared
// memory (Nyland et al., GPU Gems 3, cited at P:334); sources are split into
// chunks across blocks and the per-chunk partial sums are reduced in a fixed
// order, so results are deterministic.
#include "internal.cuh"

namespace nb {
namespace {

constexpr int kDThreads = 128;  // targets per block
constexpr int kDTile = 256;     // sources staged per iteration

// partial[chunk][t] = sum over sources j in chunk, j != slot[t], of
// m_j r / (r^2 + eps^2)^(3/2)
__global__ __launch_bounds__(kDThreads) void k_direct_partial(const float4* __restrict__ pm, int64_t n,
                                                              const uint32_t* __restrict__ tslot, int64_t nt,
                                                              double eps2, int64_t chunk, double4* __restrict__ part) {
  __shared__ float4 src[kDTile];
  const int64_t t = int64_t(blockIdx.x) * kDThreads + threadIdx.x;
  const int64_t c = blockIdx.y;
  const int64_t j0 = c * chunk, j1 = (j0 + chunk < n) ? j0 + chunk : n;
  const bool on = t < nt;
  const uint32_t self = on ? tslot[t] : 0xffffffffu;
  const float4 me = on ? pm[self] : make_float4(0.f, 0.f, 0.f, 0.f);
  const double x = me.x, y = me.y, z = me.z;
  double ax = 0.0, ay = 0.0, az = 0.0;
  for (int64_t base = j0; base < j1; base += kDTile) {
    __syncthreads();
    for (int k = threadIdx.x; k < kDTile; k += kDThreads)
      src[k] = base + k < j1 ? pm[base + k] : make_float4(0.f, 0.f, 0.f, 0.f);
    __syncthreads();
    const int cnt = int((j1 - base) < kDTile ? (j1 - base) : kDTile);
    for (int k = 0; k < cnt; ++k) {
      const float4 s = src[k];
      const double dx = double(s.x) - x, dy = double(s.y) - y, dz = double(s.z) - z;
      const double r2 = dx * dx + dy * dy + dz * dz + eps2;
      const bool use = (base + k != int64_t(self)) && r2 > 0.0;
      const double inv = use ? 1.0 / (r2 * sqrt(r2)) : 0.0;
      const double w = double(s.w) * inv;
      ax += w * dx;
      ay += w * dy;
      az += w * dz;
    }
  }
  if (on) part[c * nt + t] = make_double4(ax, ay, az, 0.0);
}

__global__ void k_direct_reduce(const double4* __restrict__ part, int64_t nt, int64_t chunks,
                                double* __restrict__ out) {
  const int64_t t = int64_t(blockIdx.x) * blockDim.x + threadIdx.x;
  if (t >= nt) return;
  double ax = 0.0, ay = 0.0, az = 0.0;
  for (int64_t c = 0; c < chunks; ++c) {
    const double4 p = part[c * nt + t];
    ax += p.x;
    ay += p.y;
    az += p.z;
  }
  out[3 * t] = ax;
  out[3 * t + 1] = ay;
  out[3 * t + 2] = az;
}

__global__ void k_slot_of_id(const float4* __restrict__ vi, int64_t n, uint32_t* __restrict__ slot_of) {
  const int64_t i = int64_t(blockIdx.x) * blockDim.x + threadIdx.x;
  if (i < n) slot_of[__float_as_int(vi[i].w)] = uint32_t(i);
}

__global__ void k_gather_u32(const uint32_t* __restrict__ table, const int64_t* __restrict__ ids, int64_t nt,
                             uint32_t* __restrict__ out) {
  const int64_t t = int64_t(blockIdx.x) * blockDim.x + threadIdx.x;
  if (t < nt) out[t] = table[ids[t]];
}

}  // namespace

int64_t direct_chunks(int64_t n, int64_t nt) {
  // enough blocks to fill the GPU several times over
  const int64_t tblocks = (nt + kDThreads - 1) / kDThreads;
  int64_t chunks = (4 * kNumSMs * 4 + tblocks - 1) / tblocks;
  if (chunks < 1) chunks = 1;
  if (chunks > 4096) chunks = 4096;
  if (chunks > n) chunks = n;
  return chunks;
}

void launch_target_slots(const float4* vi, int64_t n, const int64_t* ids, int64_t nt, uint32_t* slot_of,
                         uint32_t* tslot, cudaStream_t s) {
  if (nt <= 0) return;
  k_slot_of_id<<<unsigned((n + 255) / 256), 256, 0, s>>>(vi, n, slot_of);
  k_gather_u32<<<unsigned((nt + 255) / 256), 256, 0, s>>>(slot_of, ids, nt, tslot);
}

void launch_direct(const float4* pm, const float4* vi, int64_t n, const int64_t* ids, int64_t nt, double eps2,
                   uint32_t* slot_of, uint32_t* tslot, double4* part, double* out, cudaStream_t s) {
  if (nt <= 0) return;
  launch_target_slots(vi, n, ids, nt, slot_of, tslot, s);
  const int64_t chunks = direct_chunks(n, nt);
  const int64_t chunk = (n + chunks - 1) / chunks;
  dim3 grid(unsigned((nt + kDThreads - 1) / kDThreads), unsigned(chunks));
  k_direct_partial<<<grid, kDThreads, 0, s>>>(pm, n, tslot, nt, eps2, chunk, part);
  k_direct_reduce<<<unsigned((nt + 255) / 256), 256, 0, s>>>(part, nt, chunks, out);
}


// Load every kernel of this file now (see preload_all in capi.cu).
void preload_direct() {
  touch(k_direct_partial);
  touch(k_direct_reduce);
  touch(k_gather_u32);
  touch(k_slot_of_id);
}

}  // namespace nb
