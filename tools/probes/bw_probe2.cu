// Streaming-strategy probe (round 2): what can a kernel of each op's size and
// read/write mix get on B200, and which way of moving the bytes gets it?
//   A  grid-stride LDG/STG.128, U vectors per thread in flight, b CTAs/SM
//   B  one contiguous span per CTA, U vectors per thread per step (block-contiguous)
//   C  grid-stride LDG/STG.256 (sm_100a v8 vectors)
//   D  TMA bulk copies (cp.async.bulk global -> shared -> global), one elected
//      thread per CTA, S stages of T bytes, mbarrier-tracked loads, bulk-group stores
//   R  read-only variants of A/B/C, and D with a shared-memory sum (LDS) after each stage
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o bw_probe2 bw_probe2.cu && ./bw_probe2
// Timing: CUDA events around a batch of launches over rotating buffers (footprint > 3x L2).
#include <cstdio>
#include <cstdint>
#include <vector>
#include <functional>
#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e_ = (x); if (e_ != cudaSuccess) { printf("%s:%d %s\n", __FILE__, __LINE__, cudaGetErrorString(e_)); exit(1); } } while (0)

__device__ __forceinline__ uint4 ldg(const uint4* p) {
  uint4 v;
  asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p));
  return v;
}
struct u8v { unsigned w[8]; };
__device__ __forceinline__ u8v ldg8(const u8v* p) {
  u8v v;
  asm volatile("ld.global.nc.L1::no_allocate.v8.u32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
               : "=r"(v.w[0]), "=r"(v.w[1]), "=r"(v.w[2]), "=r"(v.w[3]), "=r"(v.w[4]), "=r"(v.w[5]), "=r"(v.w[6]), "=r"(v.w[7]) : "l"(p));
  return v;
}
__device__ __forceinline__ void stg8(u8v* p, const u8v& v) {
  asm volatile("st.global.v8.u32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8};" ::"l"(p), "r"(v.w[0]), "r"(v.w[1]), "r"(v.w[2]), "r"(v.w[3]),
               "r"(v.w[4]), "r"(v.w[5]), "r"(v.w[6]), "r"(v.w[7]) : "memory");
}

// A: grid-stride, 16 B
template <int U, bool W>
__global__ void __launch_bounds__(256) gs16(const uint4* __restrict__ in, uint4* __restrict__ out, size_t n, unsigned* sink) {
  size_t stride = (size_t)gridDim.x * blockDim.x, i = (size_t)blockIdx.x * blockDim.x + threadIdx.x;
  unsigned acc = 0;
  for (; i + (U - 1) * stride < n; i += U * stride) {
    uint4 v[U];
#pragma unroll
    for (int u = 0; u < U; ++u) v[u] = ldg(in + i + u * stride);
#pragma unroll
    for (int u = 0; u < U; ++u) { if (W) out[i + u * stride] = v[u]; else acc ^= v[u].x ^ v[u].y ^ v[u].z ^ v[u].w; }
  }
  for (; i < n; i += stride) { uint4 v = ldg(in + i); if (W) out[i] = v; else acc ^= v.x ^ v.w; }
  if (!W && acc == 0x12345678u) sink[0] = acc;
}

// B: block-contiguous span, U vectors per thread per step
template <int U, bool W>
__global__ void __launch_bounds__(256) bc16(const uint4* __restrict__ in, uint4* __restrict__ out, size_t n, unsigned* sink) {
  size_t per = (n + gridDim.x - 1) / gridDim.x;
  per = (per + 256 * U - 1) / (256 * U) * (256 * U);
  size_t s = (size_t)blockIdx.x * per, e = s + per < n ? s + per : n;
  unsigned acc = 0;
  for (size_t b = s; b < e; b += 256 * U) {
    uint4 v[U];
#pragma unroll
    for (int u = 0; u < U; ++u) { size_t i = b + u * 256 + threadIdx.x; if (i < e) v[u] = ldg(in + i); }
#pragma unroll
    for (int u = 0; u < U; ++u) {
      size_t i = b + u * 256 + threadIdx.x;
      if (i < e) { if (W) out[i] = v[u]; else acc ^= v[u].x ^ v[u].y ^ v[u].z ^ v[u].w; }
    }
  }
  if (!W && acc == 0x12345678u) sink[0] = acc;
}

// C: grid-stride, 32 B
template <int U, bool W>
__global__ void __launch_bounds__(256) gs32(const u8v* __restrict__ in, u8v* __restrict__ out, size_t n, unsigned* sink) {
  size_t stride = (size_t)gridDim.x * blockDim.x, i = (size_t)blockIdx.x * blockDim.x + threadIdx.x;
  unsigned acc = 0;
  for (; i + (U - 1) * stride < n; i += U * stride) {
    u8v v[U];
#pragma unroll
    for (int u = 0; u < U; ++u) v[u] = ldg8(in + i + u * stride);
#pragma unroll
    for (int u = 0; u < U; ++u) { if (W) stg8(out + i + u * stride, v[u]); else acc ^= v[u].w[0] ^ v[u].w[7]; }
  }
  for (; i < n; i += stride) { u8v v = ldg8(in + i); if (W) stg8(out + i, v); else acc ^= v.w[0]; }
  if (!W && acc == 0x12345678u) sink[0] = acc;
}

// D: TMA bulk copies.  Each CTA owns a contiguous span, moved in T-byte tiles
// through S shared-memory stages.  Thread 0 issues every bulk op.
__device__ __forceinline__ unsigned smem_u32(const void* p) { return (unsigned)__cvta_generic_to_shared(p); }
template <bool W>
__global__ void __launch_bounds__(128) bulk(const char* __restrict__ in, char* __restrict__ out, size_t bytes, int T, int S,
                                             unsigned* sink) {
  extern __shared__ __align__(128) char sm[];
  __shared__ __align__(8) unsigned long long bar[16];
  size_t tiles = bytes / T;
  size_t per = (tiles + gridDim.x - 1) / gridDim.x;
  size_t t0 = blockIdx.x * per, t1 = t0 + per < tiles ? t0 + per : tiles;
  if (threadIdx.x == 0)
    for (int s = 0; s < S; ++s) asm volatile("mbarrier.init.shared.b64 [%0], 1;" ::"r"(smem_u32(&bar[s])));
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  __syncthreads();
  unsigned acc = 0;
  size_t n = t1 > t0 ? t1 - t0 : 0;
  auto issue = [&](size_t k) {
    int s = k % S;
    unsigned b = smem_u32(&bar[s]);
    asm volatile("mbarrier.arrive.expect_tx.shared.b64 _, [%0], %1;" ::"r"(b), "r"(T) : "memory");
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                 ::"r"(smem_u32(sm + (size_t)s * T)), "l"(in + (t0 + k) * T), "r"(T), "r"(b) : "memory");
  };
  if (threadIdx.x == 0)
    for (size_t k = 0; k < (size_t)S && k < n; ++k) issue(k);
  for (size_t k = 0; k < n; ++k) {
    int s = k % S;
    unsigned ph = (k / S) & 1;
    unsigned b = smem_u32(&bar[s]);
    asm volatile("{ .reg .pred p; W: mbarrier.try_wait.parity.shared.b64 p, [%0], %1; @!p bra W; }" ::"r"(b), "r"(ph) : "memory");
    if (W) {
      if (threadIdx.x == 0) {
        asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(out + (t0 + k) * T),
                     "r"(smem_u32(sm + (size_t)s * T)), "r"(T) : "memory");
        asm volatile("cp.async.bulk.commit_group;" ::: "memory");
        // the stage is refilled only after its store has read it
        asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");
        if (k + S < n) issue(k + S);
      }
    } else {
      const uint4* q = (const uint4*)(sm + (size_t)s * T);
      for (int i = threadIdx.x; i < T / 16; i += blockDim.x) { uint4 v = q[i]; acc ^= v.x ^ v.w; }
      __syncthreads();
      if (threadIdx.x == 0 && k + S < n) issue(k + S);
    }
  }
  if (W && threadIdx.x == 0) asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
  if (!W && acc == 0x12345678u) sink[0] = acc;
}

struct Case { const char* name; size_t rbytes; bool write; };

int main() {
  int sms;
  CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0));
  CK(cudaFuncSetAttribute(bulk<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024));
  CK(cudaFuncSetAttribute(bulk<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024));
  Case cases[] = {
      {"read 134 MB (cfg4b)", 134217728, false},
      {"copy 50+50 MB (cfg4a)", 50331648, true},
      {"copy 411+411 MB (cfg3)", 411041792, true},
      {"copy 1+1 GiB (peak)", 1073741824, true},
      {"read 1 GiB", 1073741824, false},
  };
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  unsigned* sink;
  CK(cudaMalloc(&sink, 64));
  for (auto& c : cases) {
    int copies = (int)((400ull << 20) / c.rbytes) + 2;
    if (copies > 8) copies = 8;
    std::vector<char*> ins(copies), outs(copies);
    for (int k = 0; k < copies; ++k) {
      CK(cudaMalloc(&ins[k], c.rbytes));
      CK(cudaMemset(ins[k], k + 1, c.rbytes));
      if (c.write) CK(cudaMalloc(&outs[k], c.rbytes));
    }
    size_t tot = c.rbytes * (c.write ? 2 : 1);
    auto timeit = [&](const std::function<void(int)>& launch) {
      for (int k = 0; k < copies; ++k) launch(k);
      CK(cudaDeviceSynchronize());
      int reps = 4 * copies;
      cudaEventRecord(e0);
      for (int r = 0; r < reps; ++r) launch(r % copies);
      cudaEventRecord(e1);
      CK(cudaEventSynchronize(e1));
      float ms;
      cudaEventElapsedTime(&ms, e0, e1);
      CK(cudaGetLastError());
      return (double)tot * reps / (ms * 1e-3) / 1e9;
    };
    size_t n16 = c.rbytes / 16, n32 = c.rbytes / 32;
#define RUN(label, expr)                                                                    \
  {                                                                                         \
    double g = timeit([&](int k) { expr; });                                                \
    printf("%-26s %-34s %8.1f GB/s  %8.2f us\n", c.name, label, g, tot / g / 1e3);           \
  }
    char lab[96];
    for (int b : {2, 4, 8}) {
      int grid = sms * b;
      const uint4* i16;
      uint4* o16;
#define A(U)                                                                                                     \
  snprintf(lab, sizeof lab, "A gs16 b%d U%d", b, U);                                                             \
  RUN(lab, (i16 = (const uint4*)ins[k], o16 = (uint4*)outs[k],                                                   \
            c.write ? gs16<U, true><<<grid, 256>>>(i16, o16, n16, sink) : gs16<U, false><<<grid, 256>>>(i16, o16, n16, sink)))
      A(1) A(2) A(4) A(8)
#define B(U)                                                                                                     \
  snprintf(lab, sizeof lab, "B block-contig b%d U%d", b, U);                                                     \
  RUN(lab, (i16 = (const uint4*)ins[k], o16 = (uint4*)outs[k],                                                   \
            c.write ? bc16<U, true><<<grid, 256>>>(i16, o16, n16, sink) : bc16<U, false><<<grid, 256>>>(i16, o16, n16, sink)))
      B(2) B(4) B(8)
#define C(U)                                                                                                                  \
  snprintf(lab, sizeof lab, "C gs32 b%d U%d", b, U);                                                                          \
  RUN(lab, (c.write ? gs32<U, true><<<grid, 256>>>((const u8v*)ins[k], (u8v*)outs[k], n32, sink)                               \
                    : gs32<U, false><<<grid, 256>>>((const u8v*)ins[k], (u8v*)outs[k], n32, sink)))
      C(1) C(2) C(4)
    }
    for (int T : {8192, 16384, 32768})
      for (int S : {2, 4, 6})
        for (int b : {1, 2, 4}) {
          if ((size_t)T * S * b > 200 * 1024) continue;
          int grid = sms * b;
          snprintf(lab, sizeof lab, "D bulk T%d S%d b%d", T, S, b);
          RUN(lab, (c.write ? bulk<true><<<grid, 128, T * S>>>(ins[k], outs[k], c.rbytes, T, S, sink)
                            : bulk<false><<<grid, 128, T * S>>>(ins[k], outs[k], c.rbytes, T, S, sink)));
        }
    for (int k = 0; k < copies; ++k) {
      cudaFree(ins[k]);
      if (c.write) cudaFree(outs[k]);
    }
  }
  return 0;
}
