// Transpose probe (cfg3: NCHW [256,256,56,56] f16 -> NHWC, x 0.5): which
// global access shape gets closest to a plain copy of the same bytes?
//   A  register 8x8 tiles, warp = 8 c-tiles x 4 hw-tiles (the libfop skeleton:
//      loads 8 rows x 64 B, stores 4 rows x 128 B per warp instruction)
//   C  shared-memory staged: block tile = all C channels x 64 hw; loads 4 rows
//      x 128 B per warp instruction, stores one full 512 B NHWC row per warp
//      instruction (8x8 register transposes out of a XOR-swizzled tile)
//   copy  plain 16 B streaming copy of the same bytes (ceiling)
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tr_probe tr_probe.cu && ./tr_probe
#include <cstdio>
#include <cstdint>
#include <cstring>
#include <algorithm>
#include <vector>
#include <cuda_fp16.h>
#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e_ = (x); if (e_ != cudaSuccess) { printf("%s:%d %s\n", __FILE__, __LINE__, cudaGetErrorString(e_)); return 1; } } while (0)

constexpr int N = 256, C = 256, HW = 3136;

__device__ __forceinline__ uint4 ldg_stream(const void* p) {
  uint4 v;
  asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p));
  return v;
}
// with an L2 prefetch-size hint (PF = 128 or 256 bytes)
template <int PF>
__device__ __forceinline__ uint4 ldg_pf(const void* p) {
  uint4 v;
  if constexpr (PF == 256)
    asm volatile("ld.global.nc.L1::no_allocate.L2::256B.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p));
  else if constexpr (PF == 128)
    asm volatile("ld.global.nc.L1::no_allocate.L2::128B.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p));
  else
    v = ldg_stream(p);
  return v;
}

// 8x8 f16 transpose of rows r[0..7] (each 8 halves) scaled by s -> o[b] = column b
__device__ __forceinline__ void tr8(const uint4 (&r)[8], uint4 (&o)[8], float s) {
  float f[8][8];
#pragma unroll
  for (int a = 0; a < 8; ++a) {
    const __half2* h = reinterpret_cast<const __half2*>(&r[a]);
#pragma unroll
    for (int q = 0; q < 4; ++q) { float2 t = __half22float2(h[q]); f[a][2 * q] = t.x; f[a][2 * q + 1] = t.y; }
  }
#pragma unroll
  for (int b = 0; b < 8; ++b) {
    __half2* h = reinterpret_cast<__half2*>(&o[b]);
#pragma unroll
    for (int q = 0; q < 4; ++q) h[q] = __floats2half2_rn(f[2 * q][b] * s, f[2 * q + 1][b] * s);
  }
}

template <int U, int PF = 0>
__global__ void __launch_bounds__(256, 1) tr_A(const __half* __restrict__ x, __half* __restrict__ y, float s) {
  const unsigned tid = blockIdx.x * 256u + threadIdx.x, nth = gridDim.x * 256u;
  constexpr unsigned TRH = 98u / U;   // hw tiles of 8: 392 = TRH x U x 4
  for (unsigned g = tid; g < (unsigned)N * TRH * 4u * 4u * 8u; g += nth) {
    unsigned t = g;
    const unsigned tv_lo = t % 8u; t /= 8u;
    const unsigned tr_lo = t % 4u; t /= 4u;
    const unsigned tv_hi = t % 4u; t /= 4u;
    const unsigned tr_hi = t % TRH; t /= TRH;
    const unsigned n = t;
    const unsigned c0 = (tv_hi * 8u + tv_lo) * 8u;
    uint4 r[U][8];
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const unsigned hw0 = ((tr_hi * U + u) * 4u + tr_lo) * 8u;
#pragma unroll
      for (int a = 0; a < 8; ++a) r[u][a] = ldg_pf<PF>(x + ((size_t)n * C + c0 + a) * HW + hw0);
    }
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const unsigned hw0 = ((tr_hi * U + u) * 4u + tr_lo) * 8u;
      uint4 o[8];
      tr8(r[u], o, s);
#pragma unroll
      for (int b = 0; b < 8; ++b) *reinterpret_cast<uint4*>(y + ((size_t)n * HW + hw0 + b) * C + c0) = o[b];
    }
  }
}

// C: block tile = 256 channels x 64 hw (32 KB), smem row c = 8 chunks of 16 B, chunk j stored at j ^ ((c/8)%8)
template <int MINB>
__global__ void __launch_bounds__(256, MINB) tr_C(const __half* __restrict__ x, __half* __restrict__ y, float s) {
  __shared__ uint4 tile[C * 8];
  const unsigned t = threadIdx.x, lane = t % 32u, warp = t / 32u;
  const unsigned ntiles = N * 49u;
  for (unsigned tl = blockIdx.x; tl < ntiles; tl += gridDim.x) {
    const unsigned n = tl / 49u, hw0 = (tl % 49u) * 64u;
    uint4 v[8];
#pragma unroll
    for (int k = 0; k < 8; ++k) {
      const unsigned idx = t + 256u * k, c = idx / 8u, j = idx % 8u;
      v[k] = ldg_stream(x + ((size_t)n * C + c) * HW + hw0 + j * 8u);
    }
    __syncthreads();   // previous tile fully read out of smem
#pragma unroll
    for (int k = 0; k < 8; ++k) {
      const unsigned idx = t + 256u * k, c = idx / 8u, j = idx % 8u;
      tile[c * 8u + (j ^ ((c / 8u) % 8u))] = v[k];
    }
    __syncthreads();
    // thread: channel block lane (8 channels), hw block warp (8 hw)
    uint4 r[8], o[8];
#pragma unroll
    for (int a = 0; a < 8; ++a) {
      const unsigned c = lane * 8u + a;
      r[a] = tile[c * 8u + (warp ^ (lane % 8u))];
    }
    tr8(r, o, s);
#pragma unroll
    for (int b = 0; b < 8; ++b)
      *reinterpret_cast<uint4*>(y + ((size_t)n * HW + hw0 + warp * 8u + b) * C + lane * 8u) = o[b];
  }
}


// E: C with the next tile's global loads issued before this tile's smem read-out / stores
template <int MINB>
__global__ void __launch_bounds__(256, MINB) tr_E(const __half* __restrict__ x, __half* __restrict__ y, float s) {
  __shared__ uint4 tile[C * 8];
  const unsigned t = threadIdx.x, lane = t % 32u, warp = t / 32u;
  const unsigned ntiles = N * 49u;
  uint4 v[8];
  unsigned tl = blockIdx.x;
  auto load = [&](unsigned q) {
    const unsigned n = q / 49u, hw0 = (q % 49u) * 64u;
#pragma unroll
    for (int k = 0; k < 8; ++k) {
      const unsigned idx = t + 256u * k, c = idx / 8u, j = idx % 8u;
      v[k] = ldg_stream(x + ((size_t)n * C + c) * HW + hw0 + j * 8u);
    }
  };
  if (tl < ntiles) load(tl);
  for (; tl < ntiles; tl += gridDim.x) {
    const unsigned n = tl / 49u, hw0 = (tl % 49u) * 64u;
    __syncthreads();
#pragma unroll
    for (int k = 0; k < 8; ++k) {
      const unsigned idx = t + 256u * k, c = idx / 8u, j = idx % 8u;
      tile[c * 8u + (j ^ ((c / 8u) % 8u))] = v[k];
    }
    __syncthreads();
    if (tl + gridDim.x < ntiles) load(tl + gridDim.x);
    uint4 r[8], o[8];
#pragma unroll
    for (int a = 0; a < 8; ++a) {
      const unsigned c = lane * 8u + a;
      r[a] = tile[c * 8u + (warp ^ (lane % 8u))];
    }
    tr8(r, o, s);
#pragma unroll
    for (int b = 0; b < 8; ++b)
      *reinterpret_cast<uint4*>(y + ((size_t)n * HW + hw0 + warp * 8u + b) * C + lane * 8u) = o[b];
  }
}

__global__ void __launch_bounds__(256) copy_k(const uint4* __restrict__ in, uint4* __restrict__ out, size_t n) {
  size_t stride = (size_t)gridDim.x * blockDim.x;
  for (size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += 2 * stride) {
    uint4 a = ldg_stream(in + i), b;
    const bool two = i + stride < n;
    if (two) b = ldg_stream(in + i + stride);
    out[i] = a;
    if (two) out[i + stride] = b;
  }
}

int main() {
  int sms; CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0));
  const size_t elems = (size_t)N * C * HW, bytes = elems * 2;
  const int R = 2;
  std::vector<__half*> xs(R), ys(R);
  std::vector<__half> h(elems);
  uint32_t st = 12345;
  for (size_t i = 0; i < elems; i++) { st = st * 1664525u + 1013904223u; h[i] = __float2half(((st >> 8) & 0xffff) / 8192.f - 4.f); }
  for (int r = 0; r < R; r++) {
    CK(cudaMalloc(&xs[r], bytes)); CK(cudaMalloc(&ys[r], bytes));
    CK(cudaMemcpy(xs[r], h.data(), bytes, cudaMemcpyHostToDevice));
  }
  cudaEvent_t e0, e1; CK(cudaEventCreate(&e0)); CK(cudaEventCreate(&e1));
  auto timeit = [&](const char* name, auto launch) -> double {
    for (int i = 0; i < 3; i++) launch(i % R);
    CK(cudaDeviceSynchronize());
    double best = 1e30;
    for (int rep = 0; rep < 5; rep++) {
      const int K = 20;
      cudaEventRecord(e0);
      for (int i = 0; i < K; i++) launch(i % R);
      cudaEventRecord(e1);
      CK(cudaEventSynchronize(e1));
      float ms; cudaEventElapsedTime(&ms, e0, e1);
      best = std::min(best, (double)ms / K);
    }
    CK(cudaGetLastError());
    printf("%-28s %8.2f us  %7.1f GB/s\n", name, best * 1e3, 2.0 * bytes / (best * 1e-3) / 1e9);
    return best;
  };
  // reference result from A<1> (bitwise compare of C against it)
  std::vector<__half> ra(elems), rc(elems);
  tr_A<1><<<sms, 256>>>(xs[0], ys[0], 0.5f); CK(cudaDeviceSynchronize());
  CK(cudaMemcpy(ra.data(), ys[0], bytes, cudaMemcpyDeviceToHost));
  tr_C<4><<<sms * 4, 256>>>(xs[0], ys[1], 0.5f); CK(cudaDeviceSynchronize());
  CK(cudaMemcpy(rc.data(), ys[1], bytes, cudaMemcpyDeviceToHost));
  size_t bad = 0;
  for (size_t i = 0; i < elems; i++) bad += memcmp(&ra[i], &rc[i], 2) != 0;
  // spot-check A against the definition
  size_t badA = 0;
  for (size_t k = 0; k < 100000; k++) {
    size_t i = (k * 2654435761ull) % elems;
    size_t n = i / (C * HW), c = (i / HW) % C, p = i % HW;
    __half want = __float2half(__half2float(h[i]) * 0.5f);
    badA += memcmp(&want, &ra[(n * HW + p) * C + c], 2) != 0;
  }
  printf("A vs definition: %zu bad of 100000 sampled; C vs A: %zu bad of %zu\n", badA, bad, elems);

  timeit("copy 822 MB", [&](int r) { copy_k<<<sms * 4, 256>>>((const uint4*)xs[r], (uint4*)ys[r], bytes / 16); });
  for (int b : {1, 2})
    for (int u : {1, 2}) {
      char nm[64]; snprintf(nm, sizeof nm, "A U=%d grid=%dxSM", u, b);
      if (u == 1) timeit(nm, [&](int r) { tr_A<1><<<sms * b, 256>>>(xs[r], ys[r], 0.5f); });
      else timeit(nm, [&](int r) { tr_A<2><<<sms * b, 256>>>(xs[r], ys[r], 0.5f); });
    }
  for (int b : {2, 3, 4, 5, 6}) {
    char nm[64]; snprintf(nm, sizeof nm, "C grid=%dxSM", b);
    timeit(nm, [&](int r) {
      switch (b) {
        case 2: tr_C<2><<<sms * 2, 256>>>(xs[r], ys[r], 0.5f); break;
        case 3: tr_C<3><<<sms * 3, 256>>>(xs[r], ys[r], 0.5f); break;
        case 4: tr_C<4><<<sms * 4, 256>>>(xs[r], ys[r], 0.5f); break;
        case 5: tr_C<5><<<sms * 5, 256>>>(xs[r], ys[r], 0.5f); break;
        default: tr_C<6><<<sms * 6, 256>>>(xs[r], ys[r], 0.5f); break;
      }
    });
  }
  for (int b : {2, 3, 4}) {
    char nm[64]; snprintf(nm, sizeof nm, "E (pipelined) grid=%dxSM", b);
    timeit(nm, [&](int r) {
      switch (b) {
        case 2: tr_E<2><<<sms * 2, 256>>>(xs[r], ys[r], 0.5f); break;
        case 3: tr_E<3><<<sms * 3, 256>>>(xs[r], ys[r], 0.5f); break;
        default: tr_E<4><<<sms * 4, 256>>>(xs[r], ys[r], 0.5f); break;
      }
    });
  }
  timeit("A U=2 L2::128B", [&](int r) { tr_A<2, 128><<<sms, 256>>>(xs[r], ys[r], 0.5f); });
  timeit("A U=2 L2::256B", [&](int r) { tr_A<2, 256><<<sms, 256>>>(xs[r], ys[r], 0.5f); });
  timeit("A U=1 2xSM L2::256B", [&](int r) { tr_A<1, 256><<<sms * 2, 256>>>(xs[r], ys[r], 0.5f); });
  timeit("A U=2 (again)", [&](int r) { tr_A<2><<<sms, 256>>>(xs[r], ys[r], 0.5f); });
  tr_E<3><<<sms * 3, 256>>>(xs[0], ys[1], 0.5f); CK(cudaDeviceSynchronize());
  CK(cudaMemcpy(rc.data(), ys[1], bytes, cudaMemcpyDeviceToHost));
  bad = 0;
  for (size_t i = 0; i < elems; i++) bad += memcmp(&ra[i], &rc[i], 2) != 0;
  printf("E vs A: %zu bad\n", bad);
  timeit("copy 822 MB (again)", [&](int r) { copy_k<<<sms * 4, 256>>>((const uint4*)xs[r], (uint4*)ys[r], bytes / 16); });
  return 0;
}
