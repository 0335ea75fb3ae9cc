// cfg4a-shaped ROW_REDUCE probe (bias + GELU + row mean/var, [32768, 768] f16): the library's
// generated kernel (registers, one row prefetched per warp) vs the same row body fed by 1-D TMA bulk
// copies into a per-warp shared-memory ring of S rows (bytes in flight without registers).
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -fmad=false -I ../../paper_conf_cgo_bastoulzrlsjfjc22_b200/csrc/device \
//        -o row_tma_probe row_tma_probe.cu && ./row_tma_probe
#include <cstdio>
#include <cstdint>
#include <vector>
#include <algorithm>
#include <cuda_runtime.h>
#include <cuda_fp16.h>
#include <cstring>
#include "fop_device.cuh"
typedef unsigned idx_t;
#define CK(x) do { cudaError_t e_ = (x); if (e_ != cudaSuccess) { printf("%s:%d %s\n", __FILE__, __LINE__, cudaGetErrorString(e_)); exit(1); } } while (0)

// ---- (A) the generated kernel, verbatim (tools: FusedOp(W.cfg4a(), jit=0, autotune=0).source(0))
__global__ void __launch_bounds__(256, 3) row_reg(const FopArgs args) {
  const char* __restrict__ T0 = args.p[0];
  const char* __restrict__ T1 = args.p[1];
  char* __restrict__ T2 = args.p[2];
  char* __restrict__ T3 = args.p[3];
  char* __restrict__ T4 = args.p[4];
  const u64 fop_zero = (u64)args.zero;  (void)fop_zero;
  const idx_t lane = threadIdx.x % 32u;
  float H1[3][8];
  fop::vload<fop::F16, 8, 16, fop::LD_CACHED>(H1[0], (T1 + (u64)((unsigned)(0 + ((lane + 0u) * 8u))) * 2));
  fop::vload<fop::F16, 8, 16, fop::LD_CACHED>(H1[1], (T1 + (u64)((unsigned)(0 + ((lane + 32u) * 8u))) * 2));
  fop::vload<fop::F16, 8, 16, fop::LD_CACHED>(H1[2], (T1 + (u64)((unsigned)(0 + ((lane + 64u) * 8u))) * 2));
  u32 P0[12];
  idx_t row = ((idx_t)blockIdx.x * 256u + threadIdx.x) / 32u;
  if (row < (idx_t)32768ull) {
    idx_t pr = row;
    [[maybe_unused]] const idx_t i1_p = pr;
    fop::vload_words<fop::F16, 8, 16, fop::LD_STREAM>(&P0[0], (T0 + (u64)((unsigned)(0 + i1_p * 768 + ((lane + 0u) * 8u))) * 2));
    fop::vload_words<fop::F16, 8, 16, fop::LD_STREAM>(&P0[4], (T0 + (u64)((unsigned)(0 + i1_p * 768 + ((lane + 32u) * 8u))) * 2));
    fop::vload_words<fop::F16, 8, 16, fop::LD_STREAM>(&P0[8], (T0 + (u64)((unsigned)(0 + i1_p * 768 + ((lane + 64u) * 8u))) * 2));
  }
  #pragma unroll 1
  for (; row < (idx_t)32768ull; row += (idx_t)3552ull) {
    u32 Q0[12];
    #pragma unroll
    for (int i = 0; i < 12; ++i) Q0[i] = P0[i];
    if (row + (idx_t)3552ull < (idx_t)32768ull) {
      idx_t pr = row + (idx_t)3552ull;
      [[maybe_unused]] const idx_t i1_n = pr;
      fop::vload_words<fop::F16, 8, 16, fop::LD_STREAM>(&P0[0], (T0 + (u64)((unsigned)(0 + i1_n * 768 + ((lane + 0u) * 8u))) * 2));
      fop::vload_words<fop::F16, 8, 16, fop::LD_STREAM>(&P0[4], (T0 + (u64)((unsigned)(0 + i1_n * 768 + ((lane + 32u) * 8u))) * 2));
      fop::vload_words<fop::F16, 8, 16, fop::LD_STREAM>(&P0[8], (T0 + (u64)((unsigned)(0 + i1_n * 768 + ((lane + 64u) * 8u))) * 2));
    }
    idx_t rr = row;
    [[maybe_unused]] const idx_t i1 = rr;
    // statement 0 (ASSIGN)
    float F0[24];
    {
      [[maybe_unused]] const idx_t iv = (lane + 0u) * 8u;
      float L0[8];
      fop::cvt_words<fop::F16, 8>(L0, &Q0[0]);
      const float* L1 = H1[0];
      float R[8];
      #pragma unroll
      for (int ep = 0; ep < 4; ++ep) {
        const u64 w0_0 = fop::pk(L0[2 * ep], L0[2 * ep + 1]);
        const u64 w0_1 = fop::pk(L1[2 * ep], L1[2 * ep + 1]);
        const u64 w0_2 = fop::add2(w0_0, w0_1);
        const u64 w0_3 = fop::op_gelu_tanh2(w0_2);
        fop::upk(w0_3, R[2 * ep], R[2 * ep + 1]);
        fop::round2<fop::F16>(R[2 * ep], R[2 * ep + 1], F0[0 + 2 * ep], F0[0 + 2 * ep + 1]);
      }
      fop::vstore<fop::F16, 8, 16, fop::ST_DEFAULT>((T2 + (u64)((unsigned)(0 + i1 * 768 + iv)) * 2), R);
    }
    {
      [[maybe_unused]] const idx_t iv = (lane + 32u) * 8u;
      float L0[8];
      fop::cvt_words<fop::F16, 8>(L0, &Q0[4]);
      const float* L1 = H1[1];
      float R[8];
      #pragma unroll
      for (int ep = 0; ep < 4; ++ep) {
        const u64 w0_0 = fop::pk(L0[2 * ep], L0[2 * ep + 1]);
        const u64 w0_1 = fop::pk(L1[2 * ep], L1[2 * ep + 1]);
        const u64 w0_2 = fop::add2(w0_0, w0_1);
        const u64 w0_3 = fop::op_gelu_tanh2(w0_2);
        fop::upk(w0_3, R[2 * ep], R[2 * ep + 1]);
        fop::round2<fop::F16>(R[2 * ep], R[2 * ep + 1], F0[8 + 2 * ep], F0[8 + 2 * ep + 1]);
      }
      fop::vstore<fop::F16, 8, 16, fop::ST_DEFAULT>((T2 + (u64)((unsigned)(0 + i1 * 768 + iv)) * 2), R);
    }
    {
      [[maybe_unused]] const idx_t iv = (lane + 64u) * 8u;
      float L0[8];
      fop::cvt_words<fop::F16, 8>(L0, &Q0[8]);
      const float* L1 = H1[2];
      float R[8];
      #pragma unroll
      for (int ep = 0; ep < 4; ++ep) {
        const u64 w0_0 = fop::pk(L0[2 * ep], L0[2 * ep + 1]);
        const u64 w0_1 = fop::pk(L1[2 * ep], L1[2 * ep + 1]);
        const u64 w0_2 = fop::add2(w0_0, w0_1);
        const u64 w0_3 = fop::op_gelu_tanh2(w0_2);
        fop::upk(w0_3, R[2 * ep], R[2 * ep + 1]);
        fop::round2<fop::F16>(R[2 * ep], R[2 * ep + 1], F0[16 + 2 * ep], F0[16 + 2 * ep + 1]);
      }
      fop::vstore<fop::F16, 8, 16, fop::ST_DEFAULT>((T2 + (u64)((unsigned)(0 + i1 * 768 + iv)) * 2), R);
    }
    // statement 1 (REDUCE)
    float acc1 = 0.f;
    u64 acc1p = fop::pk1(0.f);
    {
      [[maybe_unused]] const idx_t iv = (lane + 0u) * 8u;
      #pragma unroll
      for (int ep = 0; ep < 4; ++ep) {
        const u64 w1_0 = fop::pk(F0[0 + 2 * ep], F0[0 + 2 * ep + 1]);
        acc1p = fop::add2(acc1p, w1_0);
      }
    }
    {
      [[maybe_unused]] const idx_t iv = (lane + 32u) * 8u;
      #pragma unroll
      for (int ep = 0; ep < 4; ++ep) {
        const u64 w1_0 = fop::pk(F0[8 + 2 * ep], F0[8 + 2 * ep + 1]);
        acc1p = fop::add2(acc1p, w1_0);
      }
    }
    {
      [[maybe_unused]] const idx_t iv = (lane + 64u) * 8u;
      #pragma unroll
      for (int ep = 0; ep < 4; ++ep) {
        const u64 w1_0 = fop::pk(F0[16 + 2 * ep], F0[16 + 2 * ep + 1]);
        acc1p = fop::add2(acc1p, w1_0);
      }
    }
    acc1 = __fadd_rn(acc1, __fadd_rn(fop::lo(acc1p), fop::hi(acc1p)));
    acc1 = fop::warp_sum(acc1);
    const float f1_0 = acc1;
    const float f1_1 = __uint_as_float(0x44400000u);
    const float f1_2 = __fdiv_rn(f1_0, f1_1);
    const float S1 = fop::round_to<fop::F32>(f1_2);
    if (lane == 0) fop::sstore<fop::F32>((T3 + (u64)((unsigned)(0 + i1)) * 4), f1_2);
    // statement 2 (REDUCE)
    float acc2 = 0.f;
    u64 acc2p = fop::pk1(0.f);
    {
      [[maybe_unused]] const idx_t iv = (lane + 0u) * 8u;
      const float c2_1 = S1;
      #pragma unroll
      for (int ep = 0; ep < 4; ++ep) {
        const u64 w2_0 = fop::pk(F0[0 + 2 * ep], F0[0 + 2 * ep + 1]);
        const u64 w2_2 = fop::sub2(w2_0, fop::pk1(c2_1));
        acc2p = fop::fma2(w2_2, w2_2, acc2p);
      }
    }
    {
      [[maybe_unused]] const idx_t iv = (lane + 32u) * 8u;
      const float c2_1 = S1;
      #pragma unroll
      for (int ep = 0; ep < 4; ++ep) {
        const u64 w2_0 = fop::pk(F0[8 + 2 * ep], F0[8 + 2 * ep + 1]);
        const u64 w2_2 = fop::sub2(w2_0, fop::pk1(c2_1));
        acc2p = fop::fma2(w2_2, w2_2, acc2p);
      }
    }
    {
      [[maybe_unused]] const idx_t iv = (lane + 64u) * 8u;
      const float c2_1 = S1;
      #pragma unroll
      for (int ep = 0; ep < 4; ++ep) {
        const u64 w2_0 = fop::pk(F0[16 + 2 * ep], F0[16 + 2 * ep + 1]);
        const u64 w2_2 = fop::sub2(w2_0, fop::pk1(c2_1));
        acc2p = fop::fma2(w2_2, w2_2, acc2p);
      }
    }
    acc2 = __fadd_rn(acc2, __fadd_rn(fop::lo(acc2p), fop::hi(acc2p)));
    acc2 = fop::warp_sum(acc2);
    const float f2_0 = acc2;
    const float f2_1 = __uint_as_float(0x44400000u);
    const float f2_2 = __fdiv_rn(f2_0, f2_1);
    if (lane == 0) fop::sstore<fop::F32>((T4 + (u64)((unsigned)(0 + i1)) * 4), f2_2);
  }
}


// ---- (B) TMA-fed ring: S rows of 1536 B per warp
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, unsigned bytes, u64* bar) {
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
               ::"r"(fop::smem_u32(dst)), "l"(src), "r"(bytes), "r"(fop::smem_u32(bar)) : "memory");
}
template <int S, int MINB>
__global__ void __launch_bounds__(256, MINB) row_tma(const FopArgs args) {
  const char* __restrict__ T0 = args.p[0];
  const char* __restrict__ T1 = args.p[1];
  char* __restrict__ T2 = args.p[2];
  char* __restrict__ T3 = args.p[3];
  char* __restrict__ T4 = args.p[4];
  const u64 fop_zero = (u64)args.zero;  (void)fop_zero;
  extern __shared__ __align__(128) unsigned char sm_[];
  const idx_t lane = threadIdx.x % 32u, warp = threadIdx.x / 32u;
  unsigned char* ring = sm_ + warp * (S * 1536u);
  u64* bars = (u64*)(sm_ + 8u * S * 1536u) + warp * S;
  if (lane == 0) {
    for (int s = 0; s < S; ++s) fop::mbar_init(&bars[s], 1);
    fop::fence_mbar_init();
  }
  __syncwarp();
  float H1[3][8];
  fop::vload<fop::F16, 8, 16, fop::LD_CACHED>(H1[0], (T1 + (u64)((lane + 0u) * 8u) * 2));
  fop::vload<fop::F16, 8, 16, fop::LD_CACHED>(H1[1], (T1 + (u64)((lane + 32u) * 8u) * 2));
  fop::vload<fop::F16, 8, 16, fop::LD_CACHED>(H1[2], (T1 + (u64)((lane + 64u) * 8u) * 2));
  const idx_t stride = gridDim.x * 8u;
  idx_t row = blockIdx.x * 8u + warp;
  if (lane == 0)
    for (int s = 0; s < S; ++s) {
      const idx_t r = row + s * stride;
      if (r < 32768u) { fop::mbar_expect_tx(&bars[s], 1536u); bulk_g2s(ring + s * 1536u, T0 + (u64)r * 1536u, 1536u, &bars[s]); }
    }
  #pragma unroll 1
  for (unsigned it = 0; row < 32768u; ++it, row += stride) {
    const unsigned s = it % S;
    fop::mbar_wait(&bars[s], (it / S) & 1u);
    u32 Q0[12];
    const u32 base = fop::smem_u32(ring + s * 1536u) + lane * 16u;
    fop::lds128(&Q0[0], base);
    fop::lds128(&Q0[4], base + 512u);
    fop::lds128(&Q0[8], base + 1024u);
    __syncwarp();
    if (lane == 0) {
      const idx_t rn = row + S * stride;
      if (rn < 32768u) {
        fop::fence_async_smem();
        fop::mbar_expect_tx(&bars[s], 1536u);
        bulk_g2s(ring + s * 1536u, T0 + (u64)rn * 1536u, 1536u, &bars[s]);
      }
    }
    idx_t rr = row;
    [[maybe_unused]] const idx_t i1 = rr;
    // statement 0 (ASSIGN)
    float F0[24];
    {
      [[maybe_unused]] const idx_t iv = (lane + 0u) * 8u;
      float L0[8];
      fop::cvt_words<fop::F16, 8>(L0, &Q0[0]);
      const float* L1 = H1[0];
      float R[8];
      #pragma unroll
      for (int ep = 0; ep < 4; ++ep) {
        const u64 w0_0 = fop::pk(L0[2 * ep], L0[2 * ep + 1]);
        const u64 w0_1 = fop::pk(L1[2 * ep], L1[2 * ep + 1]);
        const u64 w0_2 = fop::add2(w0_0, w0_1);
        const u64 w0_3 = fop::op_gelu_tanh2(w0_2);
        fop::upk(w0_3, R[2 * ep], R[2 * ep + 1]);
        fop::round2<fop::F16>(R[2 * ep], R[2 * ep + 1], F0[0 + 2 * ep], F0[0 + 2 * ep + 1]);
      }
      fop::vstore<fop::F16, 8, 16, fop::ST_DEFAULT>((T2 + (u64)((unsigned)(0 + i1 * 768 + iv)) * 2), R);
    }
    {
      [[maybe_unused]] const idx_t iv = (lane + 32u) * 8u;
      float L0[8];
      fop::cvt_words<fop::F16, 8>(L0, &Q0[4]);
      const float* L1 = H1[1];
      float R[8];
      #pragma unroll
      for (int ep = 0; ep < 4; ++ep) {
        const u64 w0_0 = fop::pk(L0[2 * ep], L0[2 * ep + 1]);
        const u64 w0_1 = fop::pk(L1[2 * ep], L1[2 * ep + 1]);
        const u64 w0_2 = fop::add2(w0_0, w0_1);
        const u64 w0_3 = fop::op_gelu_tanh2(w0_2);
        fop::upk(w0_3, R[2 * ep], R[2 * ep + 1]);
        fop::round2<fop::F16>(R[2 * ep], R[2 * ep + 1], F0[8 + 2 * ep], F0[8 + 2 * ep + 1]);
      }
      fop::vstore<fop::F16, 8, 16, fop::ST_DEFAULT>((T2 + (u64)((unsigned)(0 + i1 * 768 + iv)) * 2), R);
    }
    {
      [[maybe_unused]] const idx_t iv = (lane + 64u) * 8u;
      float L0[8];
      fop::cvt_words<fop::F16, 8>(L0, &Q0[8]);
      const float* L1 = H1[2];
      float R[8];
      #pragma unroll
      for (int ep = 0; ep < 4; ++ep) {
        const u64 w0_0 = fop::pk(L0[2 * ep], L0[2 * ep + 1]);
        const u64 w0_1 = fop::pk(L1[2 * ep], L1[2 * ep + 1]);
        const u64 w0_2 = fop::add2(w0_0, w0_1);
        const u64 w0_3 = fop::op_gelu_tanh2(w0_2);
        fop::upk(w0_3, R[2 * ep], R[2 * ep + 1]);
        fop::round2<fop::F16>(R[2 * ep], R[2 * ep + 1], F0[16 + 2 * ep], F0[16 + 2 * ep + 1]);
      }
      fop::vstore<fop::F16, 8, 16, fop::ST_DEFAULT>((T2 + (u64)((unsigned)(0 + i1 * 768 + iv)) * 2), R);
    }
    // statement 1 (REDUCE)
    float acc1 = 0.f;
    u64 acc1p = fop::pk1(0.f);
    {
      [[maybe_unused]] const idx_t iv = (lane + 0u) * 8u;
      #pragma unroll
      for (int ep = 0; ep < 4; ++ep) {
        const u64 w1_0 = fop::pk(F0[0 + 2 * ep], F0[0 + 2 * ep + 1]);
        acc1p = fop::add2(acc1p, w1_0);
      }
    }
    {
      [[maybe_unused]] const idx_t iv = (lane + 32u) * 8u;
      #pragma unroll
      for (int ep = 0; ep < 4; ++ep) {
        const u64 w1_0 = fop::pk(F0[8 + 2 * ep], F0[8 + 2 * ep + 1]);
        acc1p = fop::add2(acc1p, w1_0);
      }
    }
    {
      [[maybe_unused]] const idx_t iv = (lane + 64u) * 8u;
      #pragma unroll
      for (int ep = 0; ep < 4; ++ep) {
        const u64 w1_0 = fop::pk(F0[16 + 2 * ep], F0[16 + 2 * ep + 1]);
        acc1p = fop::add2(acc1p, w1_0);
      }
    }
    acc1 = __fadd_rn(acc1, __fadd_rn(fop::lo(acc1p), fop::hi(acc1p)));
    acc1 = fop::warp_sum(acc1);
    const float f1_0 = acc1;
    const float f1_1 = __uint_as_float(0x44400000u);
    const float f1_2 = __fdiv_rn(f1_0, f1_1);
    const float S1 = fop::round_to<fop::F32>(f1_2);
    if (lane == 0) fop::sstore<fop::F32>((T3 + (u64)((unsigned)(0 + i1)) * 4), f1_2);
    // statement 2 (REDUCE)
    float acc2 = 0.f;
    u64 acc2p = fop::pk1(0.f);
    {
      [[maybe_unused]] const idx_t iv = (lane + 0u) * 8u;
      const float c2_1 = S1;
      #pragma unroll
      for (int ep = 0; ep < 4; ++ep) {
        const u64 w2_0 = fop::pk(F0[0 + 2 * ep], F0[0 + 2 * ep + 1]);
        const u64 w2_2 = fop::sub2(w2_0, fop::pk1(c2_1));
        acc2p = fop::fma2(w2_2, w2_2, acc2p);
      }
    }
    {
      [[maybe_unused]] const idx_t iv = (lane + 32u) * 8u;
      const float c2_1 = S1;
      #pragma unroll
      for (int ep = 0; ep < 4; ++ep) {
        const u64 w2_0 = fop::pk(F0[8 + 2 * ep], F0[8 + 2 * ep + 1]);
        const u64 w2_2 = fop::sub2(w2_0, fop::pk1(c2_1));
        acc2p = fop::fma2(w2_2, w2_2, acc2p);
      }
    }
    {
      [[maybe_unused]] const idx_t iv = (lane + 64u) * 8u;
      const float c2_1 = S1;
      #pragma unroll
      for (int ep = 0; ep < 4; ++ep) {
        const u64 w2_0 = fop::pk(F0[16 + 2 * ep], F0[16 + 2 * ep + 1]);
        const u64 w2_2 = fop::sub2(w2_0, fop::pk1(c2_1));
        acc2p = fop::fma2(w2_2, w2_2, acc2p);
      }
    }
    acc2 = __fadd_rn(acc2, __fadd_rn(fop::lo(acc2p), fop::hi(acc2p)));
    acc2 = fop::warp_sum(acc2);
    const float f2_0 = acc2;
    const float f2_1 = __uint_as_float(0x44400000u);
    const float f2_2 = __fdiv_rn(f2_0, f2_1);
    if (lane == 0) fop::sstore<fop::F32>((T4 + (u64)((unsigned)(0 + i1)) * 4), f2_2);
  }
}

template <class K>
float time_kernel(K k, int grid, int block, size_t smem, std::vector<FopArgs>& sets) {
  cudaEvent_t a, b;
  CK(cudaEventCreate(&a)); CK(cudaEventCreate(&b));
  for (int i = 0; i < 5; ++i) k<<<grid, block, smem>>>(sets[i % sets.size()]);
  CK(cudaGetLastError()); CK(cudaDeviceSynchronize());
  std::vector<float> v;
  for (int r = 0; r < 5; ++r) {
    CK(cudaEventRecord(a));
    for (int i = 0; i < 40; ++i) k<<<grid, block, smem>>>(sets[i % sets.size()]);
    CK(cudaEventRecord(b)); CK(cudaEventSynchronize(b));
    float ms; CK(cudaEventElapsedTime(&ms, a, b)); v.push_back(ms * 1e3f / 40);
  }
  std::sort(v.begin(), v.end());
  return v[2];
}

int main() {
  const size_t R = 32768, H = 768, NX = R * H;
  const int NSET = 4;
  std::vector<FopArgs> sets(NSET);
  std::vector<uint16_t> hx(NX), hb(H);
  uint32_t st = 12345;
  auto rnd = [&]() { st = st * 1664525u + 1013904223u; return (float)((st >> 8) & 0xffff) / 65536.f * 4.f - 2.f; };
  for (auto& v : hx) { __half h = __float2half(rnd()); v = *(uint16_t*)&h; }
  for (auto& v : hb) { __half h = __float2half(rnd() * 0.05f); v = *(uint16_t*)&h; }
  char* bias; CK(cudaMalloc(&bias, H * 2)); CK(cudaMemcpy(bias, hb.data(), H * 2, cudaMemcpyHostToDevice));
  for (auto& s : sets) {
    memset(&s, 0, sizeof s);
    CK(cudaMalloc(&s.p[0], NX * 2)); CK(cudaMemcpy(s.p[0], hx.data(), NX * 2, cudaMemcpyHostToDevice));
    s.p[1] = bias;
    CK(cudaMalloc(&s.p[2], NX * 2)); CK(cudaMalloc(&s.p[3], R * 4)); CK(cudaMalloc(&s.p[4], R * 4));
  }
  const double bytes = 2.0 * NX * 2 + H * 2 + 2.0 * R * 4;
  // reference outputs from (A)
  row_reg<<<444, 256>>>(sets[0]); CK(cudaDeviceSynchronize());
  std::vector<uint16_t> ry(NX), y(NX); std::vector<float> rm(R), rv(R), m(R), vv(R);
  CK(cudaMemcpy(ry.data(), sets[0].p[2], NX * 2, cudaMemcpyDeviceToHost));
  CK(cudaMemcpy(rm.data(), sets[0].p[3], R * 4, cudaMemcpyDeviceToHost));
  CK(cudaMemcpy(rv.data(), sets[0].p[4], R * 4, cudaMemcpyDeviceToHost));
  float t = time_kernel(row_reg, 444, 256, 0, sets);
  printf("A reg (generated, 444 x 256)        %7.2f us  %6.0f GB/s\n", t, bytes / t / 1e3);
  auto runB = [&](auto kern, int S, int minb, const char* name) {
    size_t smem = 8 * S * 1536 + 8 * S * 8;
    CK(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    int grid = 148 * minb;
    CK(cudaMemset(sets[0].p[2], 0, NX * 2));
    kern<<<grid, 256, smem>>>(sets[0]); CK(cudaGetLastError()); CK(cudaDeviceSynchronize());
    CK(cudaMemcpy(y.data(), sets[0].p[2], NX * 2, cudaMemcpyDeviceToHost));
    CK(cudaMemcpy(m.data(), sets[0].p[3], R * 4, cudaMemcpyDeviceToHost));
    CK(cudaMemcpy(vv.data(), sets[0].p[4], R * 4, cudaMemcpyDeviceToHost));
    bool same = y == ry && memcmp(m.data(), rm.data(), R * 4) == 0 && memcmp(vv.data(), rv.data(), R * 4) == 0;
    float tb = time_kernel(kern, grid, 256, smem, sets);
    printf("B tma %-28s %7.2f us  %6.0f GB/s  %s\n", name, tb, bytes / tb / 1e3, same ? "bit-identical" : "MISMATCH");
  };
  runB(row_tma<2, 3>, 2, 3, "S=2 3 CTA/SM");
  runB(row_tma<3, 3>, 3, 3, "S=3 3 CTA/SM");
  runB(row_tma<4, 3>, 4, 3, "S=4 3 CTA/SM");
  runB(row_tma<6, 3>, 6, 3, "S=6 3 CTA/SM");
  runB(row_tma<2, 4>, 2, 4, "S=2 4 CTA/SM");
  runB(row_tma<3, 4>, 3, 4, "S=3 4 CTA/SM");
  runB(row_tma<4, 2>, 4, 2, "S=4 2 CTA/SM");
  runB(row_tma<8, 2>, 8, 2, "S=8 2 CTA/SM");
  t = time_kernel(row_reg, 444, 256, 0, sets);
  printf("A reg again                         %7.2f us  %6.0f GB/s\n", t, bytes / t / 1e3);
  return 0;
}
