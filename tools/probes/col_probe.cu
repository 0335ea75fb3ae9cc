// Column-sum access-pattern probe for cfg4b's shape ([65536, 1024] f16 -> f32
// column sums): which row/column decomposition lets a plain register kernel
// reach the read bandwidth the streaming probe reaches (bw_probe.cu)?
//   GV   column vectors (16 B) per block row: slab = GV*16 B
//   U    rows in flight per thread
//   B    blocks per SM (grid = SMs*B)
//   IL   0: each block owns a contiguous chunk of rows; 1: blocks interleave
//        over rows (the whole grid sweeps the matrix front to back together)
// Only the streaming part is timed (partials are written, not combined).
#include <cstdio>
#include <cstdint>
#include <vector>
#include <cuda_fp16.h>
#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e_ = (x); if (e_ != cudaSuccess) { printf("%s:%d %s\n", __FILE__, __LINE__, cudaGetErrorString(e_)); return 1; } } while (0)

constexpr int NV = 128;  // 16-byte vectors per row (1024 f16)

__device__ __forceinline__ uint4 ldg_stream(const uint4* p) {
  uint4 v;
  asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p));
  return v;
}

__device__ __forceinline__ void acc8(float* a, uint4 v) {
  const unsigned w[4] = {v.x, v.y, v.z, v.w};
#pragma unroll
  for (int i = 0; i < 4; ++i) {
    float2 f = __half22float2(*reinterpret_cast<const __half2*>(&w[i]));
    a[2 * i] += f.x;
    a[2 * i + 1] += f.y;
  }
}

template <int U, int GV, int IL>
__global__ void __launch_bounds__(256) col_k(const uint4* __restrict__ x, float* __restrict__ part, int rows) {
  constexpr int GR = 256 / GV, SLABS = NV / GV;
  const int tid = threadIdx.x, cv = tid % GV, rl = tid / GV;
  const int slab = blockIdx.x % SLABS, chunk = blockIdx.x / SLABS, nch = gridDim.x / SLABS;
  float a[8] = {0, 0, 0, 0, 0, 0, 0, 0};
  const uint4* base = x + slab * GV + cv;
  if (IL) {
    // rows r = (k*nch + chunk)*GR + rl : neighbouring chunks read neighbouring rows
    const int step = nch * GR;
    int r = chunk * GR + rl;
    for (; r + (U - 1) * step < rows; r += U * step) {
      uint4 v[U];
#pragma unroll
      for (int u = 0; u < U; ++u) v[u] = ldg_stream(base + (size_t)(r + u * step) * NV);
#pragma unroll
      for (int u = 0; u < U; ++u) acc8(a, v[u]);
    }
    for (; r < rows; r += step) acc8(a, ldg_stream(base + (size_t)r * NV));
  } else {
    const int rpc = (rows + nch - 1) / nch, r0 = chunk * rpc, r1 = min(rows, r0 + rpc);
    int r = r0 + rl;
    for (; r + (U - 1) * GR < r1; r += U * GR) {
      uint4 v[U];
#pragma unroll
      for (int u = 0; u < U; ++u) v[u] = ldg_stream(base + (size_t)(r + u * GR) * NV);
#pragma unroll
      for (int u = 0; u < U; ++u) acc8(a, v[u]);
    }
    for (; r < r1; r += GR) acc8(a, ldg_stream(base + (size_t)r * NV));
  }
  float s = 0;
#pragma unroll
  for (int e = 0; e < 8; ++e) s += a[e];
  part[(size_t)blockIdx.x * 256 + tid] = s;
}

typedef void (*KFn)(const uint4*, float*, int);

template <int U, int GV, int IL> KFn pick() { return col_k<U, GV, IL>; }

int main() {
  int sms; CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0));
  const int rows = 65536;
  const size_t bytes = (size_t)rows * NV * 16;
  const int copies = 4;
  std::vector<uint4*> xs(copies);
  for (auto& p : xs) { CK(cudaMalloc(&p, bytes)); CK(cudaMemset(p, 0x3c, bytes)); }
  float* part; CK(cudaMalloc(&part, (size_t)sms * 16 * 256 * sizeof(float)));
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  struct V { const char* n; int U, GV, IL; KFn f; };
  V vs[] = {
    {"U2 GV8 chunk", 2, 8, 0, pick<2, 8, 0>()}, {"U4 GV8 chunk", 4, 8, 0, pick<4, 8, 0>()}, {"U8 GV8 chunk", 8, 8, 0, pick<8, 8, 0>()},
    {"U2 GV8 intl", 2, 8, 1, pick<2, 8, 1>()}, {"U4 GV8 intl", 4, 8, 1, pick<4, 8, 1>()}, {"U8 GV8 intl", 8, 8, 1, pick<8, 8, 1>()},
    {"U4 GV16 chunk", 4, 16, 0, pick<4, 16, 0>()}, {"U8 GV16 chunk", 8, 16, 0, pick<8, 16, 0>()},
    {"U4 GV16 intl", 4, 16, 1, pick<4, 16, 1>()}, {"U8 GV16 intl", 8, 16, 1, pick<8, 16, 1>()},
    {"U4 GV32 chunk", 4, 32, 0, pick<4, 32, 0>()}, {"U8 GV32 chunk", 8, 32, 0, pick<8, 32, 0>()},
    {"U4 GV32 intl", 4, 32, 1, pick<4, 32, 1>()}, {"U8 GV32 intl", 8, 32, 1, pick<8, 32, 1>()},
    {"U4 GV128 chunk", 4, 128, 0, pick<4, 128, 0>()}, {"U8 GV128 chunk", 8, 128, 0, pick<8, 128, 0>()},
    {"U4 GV128 intl", 4, 128, 1, pick<4, 128, 1>()}, {"U8 GV128 intl", 8, 128, 1, pick<8, 128, 1>()},
  };
  for (auto& v : vs) {
    double best = 0; int bb = 0;
    const int slabs = NV / v.GV;
    for (int b : {1, 2, 3, 4, 6, 8}) {
      int nch = sms * b / slabs;
      if (nch < 1) continue;
      int grid = nch * slabs;
      for (int k = 0; k < copies; ++k) v.f<<<grid, 256>>>(xs[k], part, rows);
      const int reps = 24;
      cudaEventRecord(e0);
      for (int r = 0; r < reps; ++r) v.f<<<grid, 256>>>(xs[r % copies], part, rows);
      cudaEventRecord(e1); CK(cudaEventSynchronize(e1));
      float ms; cudaEventElapsedTime(&ms, e0, e1);
      double gbs = (double)bytes * reps / (ms * 1e-3) / 1e9;
      if (gbs > best) { best = gbs; bb = b; }
    }
    printf("%-16s best %7.1f GB/s (%.2f us) at %d blocks/SM\n", v.n, best, bytes / best / 1e3, bb);
  }
  return 0;
}
