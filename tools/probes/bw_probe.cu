// Achievable-bandwidth probe: plain streaming kernels at the byte counts of the
// bench ops, to tell how far each libfop kernel is from what HBM gives a kernel
// of that size and read/write mix (short kernels pay ramp-up/drain).
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o bw_probe bw_probe.cu && ./bw_probe
// Timing: CUDA events around a batch of launches over rotating buffers (total
// footprint > 3x L2), best of several configurations (grid = SMs x b, unroll U).
#include <cstdio>
#include <cstdint>
#include <vector>
#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e_ = (x); if (e_ != cudaSuccess) { printf("%s:%d %s\n", __FILE__, __LINE__, cudaGetErrorString(e_)); return 1; } } while (0)

__device__ __forceinline__ uint4 ldg_stream(const uint4* p) {
  uint4 v;
  asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p));
  return v;
}

template <int U>
__global__ void __launch_bounds__(256) read_k(const uint4* __restrict__ in, size_t n, unsigned* out) {
  size_t stride = (size_t)gridDim.x * blockDim.x;
  unsigned acc = 0;
  size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x;
  for (; i + (U - 1) * stride < n; i += U * stride) {
    uint4 v[U];
#pragma unroll
    for (int u = 0; u < U; ++u) v[u] = ldg_stream(in + i + u * stride);
#pragma unroll
    for (int u = 0; u < U; ++u) acc ^= v[u].x ^ v[u].y ^ v[u].z ^ v[u].w;
  }
  for (; i < n; i += stride) { uint4 v = ldg_stream(in + i); acc ^= v.x ^ v.y ^ v.z ^ v.w; }
  if (acc == 0x12345678u) out[0] = acc;
}

// streaming "reduce-copy": each unit reads WD adjacent vectors and writes one (WD = 1: copy, 2: cfg2's 4 B -> 2 B)
template <int U, int WD>
__global__ void __launch_bounds__(256) copy_k(const uint4* __restrict__ in, uint4* __restrict__ out, size_t n) {
  size_t stride = (size_t)gridDim.x * blockDim.x;
  size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x;
  for (; i + (U - 1) * stride < n; i += U * stride) {
    uint4 v[U][WD];
#pragma unroll
    for (int u = 0; u < U; ++u)
#pragma unroll
      for (int d = 0; d < WD; ++d) v[u][d] = ldg_stream(in + (i + u * stride) * WD + d);
#pragma unroll
    for (int u = 0; u < U; ++u) {
      uint4 w = v[u][0];
      if (WD == 2) { w.x ^= v[u][1].x; w.y ^= v[u][1].y; w.z ^= v[u][1].z; w.w ^= v[u][1].w; }
      out[i + u * stride] = w;
    }
  }
  for (; i < n; i += stride) { uint4 w = ldg_stream(in + i * WD); if (WD == 2) w.x ^= ldg_stream(in + i * WD + 1).x; out[i] = w; }
}

struct Case { const char* name; size_t rbytes; int wdiv; };  // wdiv 0 = read only; writes = rbytes / wdiv

int main() {
  int sms; CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0));
  Case cases[] = {
    {"cfg4b-like read 134 MB", 134217728, 0},
    {"cfg4a-like 50 MB read + 50 MB write", 50331648, 1},
    {"cfg2-like 411 MB read + 206 MB write", 411041792, 2},
    {"cfg3-like 411 MB read + 411 MB write", 411041792, 1},
    {"copy 1 GiB + 1 GiB", 1073741824, 1},
    {"read 411 MB", 411041792, 0},
    {"read 1 GiB", 1073741824, 0},
  };
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  unsigned* sink; CK(cudaMalloc(&sink, 64));
  for (auto& c : cases) {
    size_t n = c.wdiv ? c.rbytes / 16 / c.wdiv : c.rbytes / 16;
    size_t wbytes = c.wdiv ? c.rbytes / c.wdiv : 0;
    int copies = (int)((400ull << 20) / c.rbytes) + 2;  // rotate so the footprint exceeds 3x L2
    if (copies > 8) copies = 8;
    std::vector<void*> ins(copies), outs(copies);
    for (int k = 0; k < copies; ++k) {
      CK(cudaMalloc(&ins[k], c.rbytes)); CK(cudaMemset(ins[k], k + 1, c.rbytes));
      if (wbytes) CK(cudaMalloc(&outs[k], wbytes));
    }
    double best = 0; int bb = 0, bu = 0;
    for (int b : {1, 2, 3, 4, 6, 8}) for (int U : {1, 2, 4, 8}) {
      int grid = sms * b;
      auto launch = [&](int k) {
        const uint4* in = (const uint4*)ins[k];
        if (!c.wdiv) {
          if (U == 1) read_k<1><<<grid, 256>>>(in, n, sink); else if (U == 2) read_k<2><<<grid, 256>>>(in, n, sink);
          else if (U == 4) read_k<4><<<grid, 256>>>(in, n, sink); else read_k<8><<<grid, 256>>>(in, n, sink);
        } else {
          uint4* out = (uint4*)outs[k];
          if (c.wdiv == 1) { if (U == 1) copy_k<1, 1><<<grid, 256>>>(in, out, n); else if (U == 2) copy_k<2, 1><<<grid, 256>>>(in, out, n);
            else if (U == 4) copy_k<4, 1><<<grid, 256>>>(in, out, n); else copy_k<8, 1><<<grid, 256>>>(in, out, n); }
          else { if (U == 1) copy_k<1, 2><<<grid, 256>>>(in, out, n); else if (U == 2) copy_k<2, 2><<<grid, 256>>>(in, out, n);
            else if (U == 4) copy_k<4, 2><<<grid, 256>>>(in, out, n); else copy_k<8, 2><<<grid, 256>>>(in, out, n); }
        }
      };
      for (int k = 0; k < copies; ++k) launch(k);
      int reps = 4 * copies;
      cudaEventRecord(e0);
      for (int r = 0; r < reps; ++r) launch(r % copies);
      cudaEventRecord(e1); CK(cudaEventSynchronize(e1));
      float ms; cudaEventElapsedTime(&ms, e0, e1);
      double gbs = (double)(c.rbytes + wbytes) * reps / (ms * 1e-3) / 1e9;
      if (gbs > best) { best = gbs; bb = b; bu = U; }
    }
    printf("%-40s best %7.1f GB/s  (blocks/SM %d, U %d)  time %.2f us\n", c.name, best, bb, bu, (c.rbytes + wbytes) / best / 1e3);
    for (int k = 0; k < copies; ++k) { cudaFree(ins[k]); if (wbytes) cudaFree(outs[k]); }
  }
  return 0;
}
