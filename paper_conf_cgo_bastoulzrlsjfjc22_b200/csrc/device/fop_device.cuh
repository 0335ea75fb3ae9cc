// fop_device.cuh — hand-written sm_100a device primitives of libfop.
//
// Every kernel libfop launches is one of four skeletons (EW, TRANSPOSE,
// ROW_REDUCE, COL_REDUCE, see codegen.cpp) instantiated by the planner with
// compile-time shapes, strides and the fused expression, then compiled by
// NVRTC for sm_100a.  This header holds the pieces they are made of:
//   * explicit vector loads/stores — the "explicit vector types" of the
//     paper's backend vectorisation pass on B200:
//     LDG/STG.128 (16 B) and LDG/STG.256 (32 B, sm_100a only) issued as PTX;
//     streaming tensors bypass L1 (ld.global.nc.L1::no_allocate);
//   * exact fp16/bf16 <-> fp32 conversions (cvt.rn, packed f16x2/bf16x2);
//   * the fp32 operator set of the descriptor DAG (IEEE add/sub/mul/div/sqrt
//     via the _rn intrinsics: never contracted, bit-identical to the oracle);
//   * warp butterfly reductions (every lane gets the same bits).
// No CUDA headers: NVRTC compiles this with only its built-ins.
#pragma once

typedef unsigned int u32;
typedef unsigned short u16;
typedef unsigned long long u64;

namespace fop {

enum { F32 = 0, F16 = 1, BF16 = 2, I32 = 3 };
enum { LD_STREAM = 0, LD_CACHED = 1, LD_COHERENT = 2 };
enum { ST_DEFAULT = 0, ST_STREAM = 1 };

template <int DT> struct ES { enum { v = (DT == F16 || DT == BF16) ? 2 : 4 }; };

// ------------------------------------------------------------------ loads
template <int CB, int POL>
__device__ __forceinline__ void ldraw(u32* w, const char* p) {
  if constexpr (CB == 32) {
    if constexpr (POL == LD_STREAM)
      asm volatile("ld.global.nc.L1::no_allocate.v8.b32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
                   : "=r"(w[0]), "=r"(w[1]), "=r"(w[2]), "=r"(w[3]), "=r"(w[4]), "=r"(w[5]),
                     "=r"(w[6]), "=r"(w[7]) : "l"(p));
    else if constexpr (POL == LD_CACHED)
      asm volatile("ld.global.nc.v8.b32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
                   : "=r"(w[0]), "=r"(w[1]), "=r"(w[2]), "=r"(w[3]), "=r"(w[4]), "=r"(w[5]),
                     "=r"(w[6]), "=r"(w[7]) : "l"(p));
    else
      asm volatile("ld.global.v8.b32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
                   : "=r"(w[0]), "=r"(w[1]), "=r"(w[2]), "=r"(w[3]), "=r"(w[4]), "=r"(w[5]),
                     "=r"(w[6]), "=r"(w[7]) : "l"(p) : "memory");
  } else if constexpr (CB == 16) {
    if constexpr (POL == LD_STREAM)
      asm volatile("ld.global.nc.L1::no_allocate.v4.b32 {%0,%1,%2,%3}, [%4];"
                   : "=r"(w[0]), "=r"(w[1]), "=r"(w[2]), "=r"(w[3]) : "l"(p));
    else if constexpr (POL == LD_CACHED)
      asm volatile("ld.global.nc.v4.b32 {%0,%1,%2,%3}, [%4];"
                   : "=r"(w[0]), "=r"(w[1]), "=r"(w[2]), "=r"(w[3]) : "l"(p));
    else
      asm volatile("ld.global.v4.b32 {%0,%1,%2,%3}, [%4];"
                   : "=r"(w[0]), "=r"(w[1]), "=r"(w[2]), "=r"(w[3]) : "l"(p) : "memory");
  } else if constexpr (CB == 8) {
    if constexpr (POL == LD_STREAM)
      asm volatile("ld.global.nc.L1::no_allocate.v2.b32 {%0,%1}, [%2];" : "=r"(w[0]), "=r"(w[1]) : "l"(p));
    else if constexpr (POL == LD_CACHED)
      asm volatile("ld.global.nc.v2.b32 {%0,%1}, [%2];" : "=r"(w[0]), "=r"(w[1]) : "l"(p));
    else
      asm volatile("ld.global.v2.b32 {%0,%1}, [%2];" : "=r"(w[0]), "=r"(w[1]) : "l"(p) : "memory");
  } else {
    static_assert(CB == 4, "chunk");
    if constexpr (POL == LD_STREAM)
      asm volatile("ld.global.nc.L1::no_allocate.b32 %0, [%1];" : "=r"(w[0]) : "l"(p));
    else if constexpr (POL == LD_CACHED)
      asm volatile("ld.global.nc.b32 %0, [%1];" : "=r"(w[0]) : "l"(p));
    else
      asm volatile("ld.global.b32 %0, [%1];" : "=r"(w[0]) : "l"(p) : "memory");
  }
}

template <int POL>
__device__ __forceinline__ u16 ld16(const char* p) {
  u16 h;
  if constexpr (POL == LD_STREAM)
    asm volatile("ld.global.nc.L1::no_allocate.b16 %0, [%1];" : "=h"(h) : "l"(p));
  else if constexpr (POL == LD_CACHED)
    asm volatile("ld.global.nc.b16 %0, [%1];" : "=h"(h) : "l"(p));
  else
    asm volatile("ld.global.b16 %0, [%1];" : "=h"(h) : "l"(p) : "memory");
  return h;
}

// ------------------------------------------------------------------ stores
template <int CB, int POL>
__device__ __forceinline__ void straw(char* p, const u32* w) {
  if constexpr (CB == 32) {
    if constexpr (POL == ST_STREAM)
      asm volatile("st.global.cs.v8.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8};" ::"l"(p), "r"(w[0]), "r"(w[1]),
                   "r"(w[2]), "r"(w[3]), "r"(w[4]), "r"(w[5]), "r"(w[6]), "r"(w[7]) : "memory");
    else
      asm volatile("st.global.v8.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8};" ::"l"(p), "r"(w[0]), "r"(w[1]),
                   "r"(w[2]), "r"(w[3]), "r"(w[4]), "r"(w[5]), "r"(w[6]), "r"(w[7]) : "memory");
  } else if constexpr (CB == 16) {
    if constexpr (POL == ST_STREAM)
      asm volatile("st.global.cs.v4.b32 [%0], {%1,%2,%3,%4};" ::"l"(p), "r"(w[0]), "r"(w[1]), "r"(w[2]),
                   "r"(w[3]) : "memory");
    else
      asm volatile("st.global.v4.b32 [%0], {%1,%2,%3,%4};" ::"l"(p), "r"(w[0]), "r"(w[1]), "r"(w[2]),
                   "r"(w[3]) : "memory");
  } else if constexpr (CB == 8) {
    if constexpr (POL == ST_STREAM)
      asm volatile("st.global.cs.v2.b32 [%0], {%1,%2};" ::"l"(p), "r"(w[0]), "r"(w[1]) : "memory");
    else
      asm volatile("st.global.v2.b32 [%0], {%1,%2};" ::"l"(p), "r"(w[0]), "r"(w[1]) : "memory");
  } else {
    static_assert(CB == 4, "chunk");
    if constexpr (POL == ST_STREAM)
      asm volatile("st.global.cs.b32 [%0], %1;" ::"l"(p), "r"(w[0]) : "memory");
    else
      asm volatile("st.global.b32 [%0], %1;" ::"l"(p), "r"(w[0]) : "memory");
  }
}

__device__ __forceinline__ void st16(char* p, u16 h) {
  asm volatile("st.global.b16 [%0], %1;" ::"l"(p), "h"(h) : "memory");
}

// ------------------------------------------------------------------ conversions
__device__ __forceinline__ float h2f(u16 h) {
  float f;
  asm("cvt.f32.f16 %0, %1;" : "=f"(f) : "h"(h));
  return f;
}
__device__ __forceinline__ float b2f(u16 h) { return __uint_as_float(((u32)h) << 16); }
__device__ __forceinline__ u16 f2h(float f) {
  u16 h;
  asm("cvt.rn.f16.f32 %0, %1;" : "=h"(h) : "f"(f));
  return h;
}
__device__ __forceinline__ u16 f2b(float f) {
  u16 h;
  asm("cvt.rn.bf16.f32 %0, %1;" : "=h"(h) : "f"(f));
  return h;
}
// packed pairs: lo in bits 0..15
__device__ __forceinline__ u32 f2h2(float lo, float hi) {
  u32 r;
  asm("cvt.rn.f16x2.f32 %0, %1, %2;" : "=r"(r) : "f"(hi), "f"(lo));
  return r;
}
__device__ __forceinline__ u32 f2b2(float lo, float hi) {
  u32 r;
  asm("cvt.rn.bf16x2.f32 %0, %1, %2;" : "=r"(r) : "f"(hi), "f"(lo));
  return r;
}

template <int DT>
__device__ __forceinline__ float round_to(float v) {
  if constexpr (DT == F16) return h2f(f2h(v));
  else if constexpr (DT == BF16) return b2f(f2b(v));
  else return v;
}

// ------------------------------------------------------------------ typed vectors
// N elements of type DT at p (aligned to CB bytes) -> fp32
template <int DT, int N, int CB, int POL>
__device__ __forceinline__ void vload(float* v, const char* p) {
  constexpr int TOT = N * ES<DT>::v;
  if constexpr (CB >= 4) {
    u32 w[TOT / 4];
#pragma unroll
    for (int c = 0; c < TOT / CB; ++c) ldraw<CB, POL>(w + c * (CB / 4), p + c * CB);
#pragma unroll
    for (int i = 0; i < TOT / 4; ++i) {
      if constexpr (DT == F32 || DT == I32) {
        v[i] = __uint_as_float(w[i]);
      } else if constexpr (DT == F16) {
        v[2 * i] = h2f((u16)(w[i] & 0xffffu));
        v[2 * i + 1] = h2f((u16)(w[i] >> 16));
      } else {
        v[2 * i] = __uint_as_float(w[i] << 16);
        v[2 * i + 1] = __uint_as_float(w[i] & 0xffff0000u);
      }
    }
  } else {
#pragma unroll
    for (int i = 0; i < N; ++i) {
      u16 h = ld16<POL>(p + 2 * i);
      v[i] = DT == F16 ? h2f(h) : b2f(h);
    }
  }
}

// split form of vload for software prefetch: raw words now, conversion later
template <int DT, int N, int CB, int POL>
__device__ __forceinline__ void vload_words(u32* w, const char* p) {
  constexpr int TOT = N * ES<DT>::v;
  static_assert(CB >= 4 && TOT % CB == 0, "word-granular vectors only");
#pragma unroll
  for (int c = 0; c < TOT / CB; ++c) ldraw<CB, POL>(w + c * (CB / 4), p + c * CB);
}
template <int DT, int N>
__device__ __forceinline__ void cvt_words(float* v, const u32* w) {
  constexpr int TOT = N * ES<DT>::v;
#pragma unroll
  for (int i = 0; i < TOT / 4; ++i) {
    if constexpr (DT == F32 || DT == I32) {
      v[i] = __uint_as_float(w[i]);
    } else if constexpr (DT == F16) {
      v[2 * i] = h2f((u16)(w[i] & 0xffffu));
      v[2 * i + 1] = h2f((u16)(w[i] >> 16));
    } else {
      v[2 * i] = __uint_as_float(w[i] << 16);
      v[2 * i + 1] = __uint_as_float(w[i] & 0xffff0000u);
    }
  }
}

// fp32 -> N elements of type DT at p (RNE conversion)
template <int DT, int N, int CB, int POL>
__device__ __forceinline__ void vstore(char* p, const float* v) {
  constexpr int TOT = N * ES<DT>::v;
  if constexpr (CB >= 4) {
    u32 w[TOT / 4];
#pragma unroll
    for (int i = 0; i < TOT / 4; ++i) {
      if constexpr (DT == F32 || DT == I32) w[i] = __float_as_uint(v[i]);
      else if constexpr (DT == F16) w[i] = f2h2(v[2 * i], v[2 * i + 1]);
      else w[i] = f2b2(v[2 * i], v[2 * i + 1]);
    }
#pragma unroll
    for (int c = 0; c < TOT / CB; ++c) straw<CB, POL>(p + c * CB, w + c * (CB / 4));
  } else {
#pragma unroll
    for (int i = 0; i < N; ++i) st16(p + 2 * i, DT == F16 ? f2h(v[i]) : f2b(v[i]));
  }
}

// raw element moves (pure copies/transposes keep every bit, NaN payloads too)
template <int ESZ, int N, int CB, int POL>
__device__ __forceinline__ void vload_raw(u32* e, const char* p) {  // one element per u32
  constexpr int TOT = N * ESZ;
  if constexpr (CB >= 4) {
    u32 w[TOT / 4];
#pragma unroll
    for (int c = 0; c < TOT / CB; ++c) ldraw<CB, POL>(w + c * (CB / 4), p + c * CB);
#pragma unroll
    for (int i = 0; i < TOT / 4; ++i) {
      if constexpr (ESZ == 4) {
        e[i] = w[i];
      } else {
        e[2 * i] = w[i] & 0xffffu;
        e[2 * i + 1] = w[i] >> 16;
      }
    }
  } else {
#pragma unroll
    for (int i = 0; i < N; ++i) e[i] = ld16<POL>(p + 2 * i);
  }
}

template <int ESZ, int N, int CB, int POL>
__device__ __forceinline__ void vstore_raw(char* p, const u32* e) {
  constexpr int TOT = N * ESZ;
  if constexpr (CB >= 4) {
    u32 w[TOT / 4];
#pragma unroll
    for (int i = 0; i < TOT / 4; ++i) {
      if constexpr (ESZ == 4) w[i] = e[i];
      else w[i] = (e[2 * i] & 0xffffu) | (e[2 * i + 1] << 16);
    }
#pragma unroll
    for (int c = 0; c < TOT / CB; ++c) straw<CB, POL>(p + c * CB, w + c * (CB / 4));
  } else {
#pragma unroll
    for (int i = 0; i < N; ++i) st16(p + 2 * i, (u16)e[i]);
  }
}

template <int DT, int POL>
__device__ __forceinline__ float sload(const char* p) {
  if constexpr (DT == F32 || DT == I32) {
    u32 w;
    ldraw<4, POL>(&w, p);
    return __uint_as_float(w);
  } else {
    u16 h = ld16<POL>(p);
    return DT == F16 ? h2f(h) : b2f(h);
  }
}

template <int DT>
__device__ __forceinline__ void sstore(char* p, float v) {
  if constexpr (DT == F32 || DT == I32) {
    u32 w = __float_as_uint(v);
    straw<4, ST_DEFAULT>(p, &w);
  } else {
    st16(p, DT == F16 ? f2h(v) : f2b(v));
  }
}

template <int ESZ, int POL>
__device__ __forceinline__ u32 sload_raw(const char* p) {
  if constexpr (ESZ == 4) {
    u32 w;
    ldraw<4, POL>(&w, p);
    return w;
  } else {
    return ld16<POL>(p);
  }
}

template <int ESZ>
__device__ __forceinline__ void sstore_raw(char* p, u32 e) {
  if constexpr (ESZ == 4) straw<4, ST_DEFAULT>(p, &e);
  else st16(p, (u16)e);
}

// ------------------------------------------------------------------ operators
// fp32 semantics shared with the oracle (include/fop.h); + - * / sqrt are the
// _rn intrinsics, which the compiler never fuses into FMA.
__device__ __forceinline__ float op_relu(float a) { return a > 0.f ? a : 0.f; }
// max/min: NaN operands ignored, max(-0,+0) = +0, min(-0,+0) = -0 (reading
// R24).  B200's FMNMX implements exactly this (tools/probes/maxmin_probe.cu,
// measured), so fmaxf/fminf are single instructions with the oracle's bits.
// Written as PTX min/max (the same FMNMX fminf/fmaxf compile to): CUDA 12.9's
// NVVM optimizer crashes the compiling process (SIGILL inside cicc/NVRTC) on
// min(min(a, b), a + b) and max(max(a, b), a * b) built from the intrinsics
// (fuzz seed 15 case 161; tools/probes/cicc_minmax.cu); inline PTX is opaque
// to that rewrite.
__device__ __forceinline__ float op_max(float a, float b) {
  float r;
  asm("max.f32 %0, %1, %2;" : "=f"(r) : "f"(a), "f"(b));
  return r;
}
__device__ __forceinline__ float op_min(float a, float b) {
  float r;
  asm("min.f32 %0, %1, %2;" : "=f"(r) : "f"(a), "f"(b));
  return r;
}
// .ftz forms: MUFU.EX2/RCP without the subnormal pre/post scaling.  In GELU
// the flushed cases are e < 2^-126 (1 + e == 1 either way) and results below
// 2^-126 (below fp16/bf16 resolution by 2^-100).
__device__ __forceinline__ float ex2_approx(float x) {
  float r;
  asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(r) : "f"(x));
  return r;
}
__device__ __forceinline__ float rcp_approx(float x) {
  float r;
  asm("rcp.approx.ftz.f32 %0, %1;" : "=f"(r) : "f"(x));
  return r;
}

// ------------------------------------------------------------------ packed fp32x2
// sm_100a executes add/sub/mul/fma on register pairs (FADD2/FMUL2/FFMA2):
// half the instructions per element, each lane IEEE round-to-nearest exactly
// like the scalar op (bit-identical results).
__device__ __forceinline__ u64 pk(float a, float b) {
  u64 r;
  asm("mov.b64 %0, {%1, %2};" : "=l"(r) : "f"(a), "f"(b));
  return r;
}
__device__ __forceinline__ u64 pk1(float a) { return pk(a, a); }
__device__ __forceinline__ void upk(u64 v, float& a, float& b) {
  asm("mov.b64 {%0, %1}, %2;" : "=f"(a), "=f"(b) : "l"(v));
}
__device__ __forceinline__ float lo(u64 v) {
  float a, b;
  upk(v, a, b);
  return a;
}
__device__ __forceinline__ float hi(u64 v) {
  float a, b;
  upk(v, a, b);
  return b;
}
__device__ __forceinline__ u64 add2(u64 a, u64 b) {
  u64 r;
  asm("add.rn.f32x2 %0, %1, %2;" : "=l"(r) : "l"(a), "l"(b));
  return r;
}
__device__ __forceinline__ u64 sub2(u64 a, u64 b) {
  u64 r;
  asm("sub.rn.f32x2 %0, %1, %2;" : "=l"(r) : "l"(a), "l"(b));
  return r;
}
__device__ __forceinline__ u64 mul2(u64 a, u64 b) {
  u64 r;
  asm("mul.rn.f32x2 %0, %1, %2;" : "=l"(r) : "l"(a), "l"(b));
  return r;
}
// ptxas (12.9, -O3) contracts mul.rn.f32x2 feeding add.rn.f32x2 into FFMA2
// even under -fmad=false, which would change the rounding.  OR-ing the
// product with a zero ptxas cannot prove hides the pattern at the cost of one
// integer op per pair.  The zero is FopArgs::zero, a kernel parameter the
// runtime always sets to 0 (round 2 used %dynamic_smem_size, which is NOT zero
// in the kernels launched with dynamic shared memory — the TMA transposes —
// and corrupted their products once every product was hidden).
__device__ __forceinline__ u64 nofuse(u64 v, u64 zero) { return v | zero; }
__device__ __forceinline__ u64 fma2(u64 a, u64 b, u64 c) {
  u64 r;
  asm("fma.rn.f32x2 %0, %1, %2, %3;" : "=l"(r) : "l"(a), "l"(b), "l"(c));
  return r;
}

// a / d for a pair by a loop-invariant d: q0 = RN(a r) with r = RN(1/d),
// remainder rem = RN(a - q0 d) by FMA, q = RN(q0 + rem r).  With r the
// correctly rounded reciprocal and q0 within one ulp of a/d this is
// Markstein's correction: q == RN(a/d), the same bits as __fdiv_rn
// (tests/test_fastdiv.py checks the formula against exact rational division).
// Outside the range where the theorem's premises hold the lane takes
// __fdiv_rn itself: d zero, subnormal, huge, inf or NaN (r not a normal
// number: uniform over the launch, d is invariant); a quotient that overflows,
// underflows or is not a number (q0 outside [2^-100, FLT_MAX]); a dividend
// below 2^-100 (its remainder would be subnormal, hence inexact); a = +-0 keeps
// q0 (the correction would turn -0 into +0).
__device__ __forceinline__ bool div_by_ok(float d) { return fabsf(d) >= 0x1p-125f && fabsf(d) <= 0x1p125f; }
__device__ __forceinline__ float div_by_fix(float q, float q0, float a, float d) {
  const float m = fabsf(q0);
  if (m >= 0x1p-100f && m <= 0x1.fffffep127f && fabsf(a) >= 0x1p-100f) return q;
  return a == 0.0f ? q0 : __fdiv_rn(a, d);
}
__device__ __forceinline__ u64 div2_by(u64 a, float d) {
  if (!div_by_ok(d)) return pk(__fdiv_rn(lo(a), d), __fdiv_rn(hi(a), d));
  const float r = __frcp_rn(d);
  const u64 q0 = mul2(a, pk1(r));
  const u64 rem = fma2(q0, pk1(-d), a);
  const u64 q = fma2(rem, pk1(r), q0);
  const float m0 = fabsf(lo(q0)), m1 = fabsf(hi(q0));
  const float a0 = fabsf(lo(a)), a1 = fabsf(hi(a));
  if (fminf(fminf(m0, m1), fminf(a0, a1)) >= 0x1p-100f && fmaxf(m0, m1) <= 0x1.fffffep127f) return q;
  return pk(div_by_fix(lo(q), lo(q0), lo(a), d), div_by_fix(hi(q), hi(q0), hi(a), d));
}

// ------------------------------------------------------------------ int32 (reading R30)
// Integer statements keep int32 values as raw bits in the same 32-bit
// registers the fp32 DAG uses (loads/stores of I32 move raw bits); their
// nodes operate on those bits with two's-complement wrap-around (unsigned
// arithmetic modulo 2^32 — no signed-overflow UB in the C++ source).
__device__ __forceinline__ float iadd(float a, float b) { return __uint_as_float(__float_as_uint(a) + __float_as_uint(b)); }
__device__ __forceinline__ float isub(float a, float b) { return __uint_as_float(__float_as_uint(a) - __float_as_uint(b)); }
__device__ __forceinline__ float imul(float a, float b) { return __uint_as_float(__float_as_uint(a) * __float_as_uint(b)); }
__device__ __forceinline__ float imax(float a, float b) { return __int_as_float(max(__float_as_int(a), __float_as_int(b))); }
__device__ __forceinline__ float imin(float a, float b) { return __int_as_float(min(__float_as_int(a), __float_as_int(b))); }
__device__ __forceinline__ float ineg(float a) { return __uint_as_float(0u - __float_as_uint(a)); }
__device__ __forceinline__ float iabs(float a) { return __float_as_int(a) < 0 ? ineg(a) : a; }
__device__ __forceinline__ float irelu(float a) { return __float_as_int(a) > 0 ? a : __int_as_float(0); }

// GELU, tanh form: 0.5 v (1 + tanh u) == v * sigmoid(2u) = v / (1 + 2^(v * (C2 + C1 v^2)))
// with u = sqrt(2/pi)(v + 0.044715 v^3), C2 = -2 sqrt(2/pi) log2(e), C1 = 0.044715 C2.
// MUFU.EX2 + MUFU.RCP: relative error ~1e-6, far inside one fp16/bf16 ulp
// (the <= 1 ulp lemma); the precise tanhf form costs ~4x the
// ALU work and would make cfg4a ALU-bound on B200.
#define FOP_GELU_C2 (-2.0f * 0.7978845608028654f * 1.4426950408889634f)
#define FOP_GELU_C1 (0.044715f * FOP_GELU_C2)
__device__ __forceinline__ float op_gelu_tanh(float v) {
  float t = fmaf(v * v, FOP_GELU_C1, FOP_GELU_C2);
  float e = ex2_approx(t * v);
  return v * rcp_approx(1.0f + e);
}
#ifndef FOP_GELU_NR
#define FOP_GELU_NR 0
#endif
__device__ __forceinline__ u64 op_gelu_tanh2(u64 v) {
  u64 t = fma2(mul2(v, v), pk1(FOP_GELU_C1), pk1(FOP_GELU_C2));
  u64 a = mul2(t, v);
#if FOP_GELU_NR
  // 1/(1+e) on the FMA pipe: MUFU.EX2 only (the XU pipe is the cfg4a limiter).
  // Clamp the exponent so 1+e stays below 2^127 (the magic-constant seed needs
  // a finite input; 1/(1+2^126) vs 0 is below fp16/bf16 resolution), seed by
  // the integer reciprocal trick, three Newton steps y <- y (2 - d y).
  u64 e = pk(ex2_approx(fminf(lo(a), 126.f)), ex2_approx(fminf(hi(a), 126.f)));
  u64 dn = add2(e, pk1(1.0f));
  u64 y = 0x7EF311C37EF311C3ull - dn;
  u64 nd = dn ^ 0x8000000080000000ull;
  y = mul2(y, fma2(nd, y, pk1(2.0f)));
  y = mul2(y, fma2(nd, y, pk1(2.0f)));
  y = mul2(y, fma2(nd, y, pk1(2.0f)));
  return mul2(v, y);
#else
  u64 e = pk(ex2_approx(lo(a)), ex2_approx(hi(a)));
  u64 dn = add2(e, pk1(1.0f));
  return mul2(v, pk(rcp_approx(lo(dn)), rcp_approx(hi(dn))));
#endif
}

// GELU for bf16 and fp32 results: their range reaches down to 2^-133 / 2^-149,
// where v / (1 + 2^a) overflows 2^a (a > 128) and the .ftz forms flush.  With
// e = 2^-|a| <= 1 (never overflows; subnormal e kept by the non-ftz ex2):
// 1 / (1 + 2^a) = (a > 0 ? e : 1) / (1 + e).  Same MUFU count; f16 results
// (whose smallest subnormal is 2^-24) keep the shorter form above.
__device__ __forceinline__ float ex2_approx_sub(float x) {
  float r;
  asm("ex2.approx.f32 %0, %1;" : "=f"(r) : "f"(x));
  return r;
}
__device__ __forceinline__ float op_gelu_tanh_wide(float v) {
  const float a = __fmul_rn(fmaf(v * v, FOP_GELU_C1, FOP_GELU_C2), v);
  const float e = ex2_approx_sub(-fabsf(a));
  const float r = rcp_approx(1.0f + e);
  return __fmul_rn(v, a > 0.0f ? __fmul_rn(e, r) : r);
}
__device__ __forceinline__ u64 op_gelu_tanh2_wide(u64 v) {
  return pk(op_gelu_tanh_wide(lo(v)), op_gelu_tanh_wide(hi(v)));
}

// value rounded to DT and back, for a pair; the packed conversion is the same
// instruction the vector store issues, so the compiler computes it once
template <int DT>
__device__ __forceinline__ void round2(float a, float b, float& ra, float& rb) {
  if constexpr (DT == F16) {
    u32 w = f2h2(a, b);
    ra = h2f((u16)(w & 0xffffu));
    rb = h2f((u16)(w >> 16));
  } else if constexpr (DT == BF16) {
    u32 w = f2b2(a, b);
    ra = __uint_as_float(w << 16);
    rb = __uint_as_float(w & 0xffff0000u);
  } else {
    ra = a;
    rb = b;
  }
}
// GELU, erf form: 0.5 v (1 + erf(v / sqrt 2)) = v Phi(v).  normcdff evaluates Phi
// without first rounding v / sqrt 2 to fp32 (an erfcf(-v * 0.7071f) form
// amplifies that rounding by ~v^2 in the negative tail); CUDA documents it to
// 5 ulp over the whole range, so v * normcdff(v) is within 6 fp32 ulp
// (tests/test_transcendental_gpu.py).
__device__ __forceinline__ float op_gelu_erf(float v) { return __fmul_rn(v, normcdff(v)); }
__device__ __forceinline__ float op_sigmoid(float v) { return __frcp_rn(1.0f + expf(-v)); }

// Fast forms, used only for statements whose result is rounded to fp16/bf16
// (DESIGN.md §4): relative error before the final rounding ~|x|*2^-24 + 2^-22
// for |x| < 100 — far below 2^-11, so the <= 1 ulp lemma holds.
__device__ __forceinline__ float exp_fast(float x) { return ex2_approx(x * 1.4426950408889634f); }
__device__ __forceinline__ float sigmoid_fast(float x) {
  return rcp_approx(1.0f + ex2_approx(x * -1.4426950408889634f));
}
// bf16 results reach down to 2^-133: no flush to zero, no 2^|x| overflow
// (the GELU wide form's identity 1 / (1 + e^-x) = (x < 0 ? e : 1) / (1 + e), e = e^-|x|)
__device__ __forceinline__ float exp_fast_wide(float x) { return ex2_approx_sub(x * 1.4426950408889634f); }
__device__ __forceinline__ float sigmoid_fast_wide(float x) {
  const float e = ex2_approx_sub(fabsf(x) * -1.4426950408889634f);
  const float r = rcp_approx(1.0f + e);
  return x < 0.0f ? e * r : r;
}

// ------------------------------------------------------------------ reductions
__device__ __forceinline__ float warp_sum(float v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v = __fadd_rn(v, __shfl_xor_sync(0xffffffffu, v, o));
  return v;
}
__device__ __forceinline__ float warp_max(float v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v = op_max(v, __shfl_xor_sync(0xffffffffu, v, o));
  return v;
}
// int32 reductions (reading R30): wrap-around sums are exactly associative,
// so every association order gives the oracle's bits
__device__ __forceinline__ float warp_isum(float v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v = iadd(v, __shfl_xor_sync(0xffffffffu, v, o));
  return v;
}
__device__ __forceinline__ float warp_imax(float v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v = imax(v, __shfl_xor_sync(0xffffffffu, v, o));
  return v;
}
template <int LN>
__device__ __forceinline__ float group_isum(float v) {
#pragma unroll
  for (int o = LN / 2; o > 0; o >>= 1) v = iadd(v, __shfl_xor_sync(0xffffffffu, v, o));
  return v;
}
template <int LN>
__device__ __forceinline__ float group_imax(float v) {
#pragma unroll
  for (int o = LN / 2; o > 0; o >>= 1) v = imax(v, __shfl_xor_sync(0xffffffffu, v, o));
  return v;
}
// butterflies over aligned groups of LN lanes (LN rows of a short-row kernel
// share a warp: the xor offsets < LN never leave the group)
template <int LN>
__device__ __forceinline__ float group_sum(float v) {
#pragma unroll
  for (int o = LN / 2; o > 0; o >>= 1) v = __fadd_rn(v, __shfl_xor_sync(0xffffffffu, v, o));
  return v;
}
template <int LN>
__device__ __forceinline__ float group_max(float v) {
#pragma unroll
  for (int o = LN / 2; o > 0; o >>= 1) v = op_max(v, __shfl_xor_sync(0xffffffffu, v, o));
  return v;
}

// ------------------------------------------------------------------ TMA + mbarrier (sm_90+/sm_100a)
// Tensor maps are encoded on the host per run (cuTensorMapEncodeTiled) and
// passed as __grid_constant__ kernel parameters.
struct alignas(64) TmaDesc {
  u64 w[16];
};
__device__ __forceinline__ u32 smem_u32(const void* p) { return (u32)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(u64* bar, u32 count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void fence_mbar_init() { asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory"); }
__device__ __forceinline__ void mbar_expect_tx(u64* bar, u32 bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes) : "memory");
}
__device__ __forceinline__ bool mbar_try(u64* bar, u32 phase) {
  u32 ok;
  asm volatile(
      "{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0, 1, 0, p; }"
      : "=r"(ok) : "r"(smem_u32(bar)), "r"(phase) : "memory");
  return ok != 0;
}
__device__ __forceinline__ void mbar_wait(u64* bar, u32 phase) {
  while (!mbar_try(bar, phase)) {
  }
}
// Arrival counter with acquire-release semantics at GPU scope: one
// atomic carries the release of the CTA's partial stores (ordered before it by
// bar.sync, release is cumulative) and the acquire of the other CTAs' (for the
// last arrival), instead of membar.gl in every thread plus a relaxed atomic.
__device__ __forceinline__ unsigned atom_add_acq_rel_gpu(unsigned* p, unsigned v) {
  unsigned old;
  asm volatile("atom.acq_rel.gpu.global.add.u32 %0, [%1], %2;" : "=r"(old) : "l"(p), "r"(v) : "memory");
  return old;
}
__device__ __forceinline__ void fence_async_smem() { asm volatile("fence.proxy.async.shared::cta;" ::: "memory"); }
__device__ __forceinline__ void bulk_commit() { asm volatile("cp.async.bulk.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void bulk_wait_read() {
  asm volatile("cp.async.bulk.wait_group.read %0;" ::"n"(N) : "memory");
}
template <int N>
__device__ __forceinline__ void bulk_wait() {
  asm volatile("cp.async.bulk.wait_group %0;" ::"n"(N) : "memory");
}
// tile loads / stores, rank 2..5 (c0 = innermost coordinate, in elements)
__device__ __forceinline__ void tma_load(void* dst, const TmaDesc* d, u64* bar, int r, const int* c) {
  u32 s = smem_u32(dst), b = smem_u32(bar);
  u64 g = (u64)d;
  if (r == 2)
    asm volatile("cp.async.bulk.tensor.2d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];"
                 ::"r"(s), "l"(g), "r"(c[0]), "r"(c[1]), "r"(b) : "memory");
  else if (r == 3)
    asm volatile("cp.async.bulk.tensor.3d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4}], [%5];"
                 ::"r"(s), "l"(g), "r"(c[0]), "r"(c[1]), "r"(c[2]), "r"(b) : "memory");
  else if (r == 4)
    asm volatile("cp.async.bulk.tensor.4d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4, %5}], [%6];"
                 ::"r"(s), "l"(g), "r"(c[0]), "r"(c[1]), "r"(c[2]), "r"(c[3]), "r"(b) : "memory");
  else
    asm volatile("cp.async.bulk.tensor.5d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4, %5, %6}], [%7];"
                 ::"r"(s), "l"(g), "r"(c[0]), "r"(c[1]), "r"(c[2]), "r"(c[3]), "r"(c[4]), "r"(b) : "memory");
}
__device__ __forceinline__ void tma_store(const TmaDesc* d, const void* src, int r, const int* c) {
  u32 s = smem_u32(src);
  u64 g = (u64)d;
  if (r == 2)
    asm volatile("cp.async.bulk.tensor.2d.global.shared::cta.tile.bulk_group [%0, {%2, %3}], [%1];"
                 ::"l"(g), "r"(s), "r"(c[0]), "r"(c[1]) : "memory");
  else if (r == 3)
    asm volatile("cp.async.bulk.tensor.3d.global.shared::cta.tile.bulk_group [%0, {%2, %3, %4}], [%1];"
                 ::"l"(g), "r"(s), "r"(c[0]), "r"(c[1]), "r"(c[2]) : "memory");
  else if (r == 4)
    asm volatile("cp.async.bulk.tensor.4d.global.shared::cta.tile.bulk_group [%0, {%2, %3, %4, %5}], [%1];"
                 ::"l"(g), "r"(s), "r"(c[0]), "r"(c[1]), "r"(c[2]), "r"(c[3]) : "memory");
  else
    asm volatile("cp.async.bulk.tensor.5d.global.shared::cta.tile.bulk_group [%0, {%2, %3, %4, %5, %6}], [%1];"
                 ::"l"(g), "r"(s), "r"(c[0]), "r"(c[1]), "r"(c[2]), "r"(c[3]), "r"(c[4]) : "memory");
}
__device__ __forceinline__ void lds128(u32* w, u32 addr) {
  asm volatile("ld.shared.v4.b32 {%0,%1,%2,%3}, [%4];" : "=r"(w[0]), "=r"(w[1]), "=r"(w[2]), "=r"(w[3]) : "r"(addr));
}
__device__ __forceinline__ void sts128(u32 addr, u32 a, u32 b, u32 c, u32 d) {
  asm volatile("st.shared.v4.b32 [%0], {%1,%2,%3,%4};" ::"r"(addr), "r"(a), "r"(b), "r"(c), "r"(d) : "memory");
}

// ---------------------------------------------------------------- thread-block clusters
// ROW_REDUCE with Q CTAs per row: block partials combined through
// distributed shared memory (every CTA reads rank 0..Q-1 in order).
__device__ __forceinline__ unsigned cluster_ctarank() {
  unsigned r;
  asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
  return r;
}
__device__ __forceinline__ void cluster_sync() {
  asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}
__device__ __forceinline__ float ld_dsmem(const float* p, unsigned rank) {
  u32 a = (u32)__cvta_generic_to_shared(p), r;
  asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(r) : "r"(a), "r"(rank));
  float v;
  asm volatile("ld.shared::cluster.f32 %0, [%1];" : "=f"(v) : "r"(r) : "memory");
  return v;
}

// ---------------------------------------------------------------- programmatic dependent launch
// Explicit PDL control, emitted only with FOP_PDL_EMIT (ablation): bit 1 =
// trigger dependents (at block end, or at start with FOP_PDL_POS=0), bit 2 =
// wait for the predecessor before completing.  Measured on the bench suite
// (tools/pdl_time.py): 357 us/step with them vs 277 us without — a dependent
// grid that launches early competes with the primary's statically
// partitioned one-wave grid — so by default kernels carry neither and
// fop_run_many's launches only get programmatic stream serialization, whose
// implicit trigger at the primary's completion keeps stream order while the
// dependent's launch is processed early.
__device__ __forceinline__ void pdl_trigger() { asm volatile("griddepcontrol.launch_dependents;" ::: "memory"); }
__device__ __forceinline__ void pdl_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }

// ---------------------------------------------------------------- peer exchange (multi-GPU)
// Cross-GPU reduction in a COL_REDUCE epilogue (fop.h, peer groups): each
// partial sum travels as ONE 64-bit word (fp32 bits | epoch << 32) stored
// into the receiver's exchange buffer over NVLink.  An aligned 64-bit
// access is single-copy atomic, so a receiver that reads the current epoch
// in the high half has the matching sum in the low half: the epoch is the
// arrival flag (no separate flag store, fence or release/acquire round trip).
__device__ __forceinline__ void st_relaxed_sys_u64(u64* p, u64 v) {
  asm volatile("st.relaxed.sys.global.b64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ u64 ld_relaxed_sys_u64(const u64* p) {
  u64 v;
  asm volatile("ld.relaxed.sys.global.b64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_relaxed_gpu_u64(u64* p, u64 v) {
  asm volatile("st.relaxed.gpu.global.b64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ u64 ld_relaxed_gpu_u64(const u64* p) {
  u64 v;
  asm volatile("ld.relaxed.gpu.global.b64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
// COL_REDUCE flag words: (1 << 32 | fp32 bits).  Poll until the valid half is
// set; the word carries the value, so no fence or atomic orders it.
// A word that never arrives (a launch that broke the one-wave residency the
// geometry guarantees) gives NaN after ~4 s instead of a hang.
__device__ __forceinline__ float wait_flag_word(const u64* p) {
  u64 w = ld_relaxed_gpu_u64(p);
  if ((unsigned)(w >> 32) != 0u) return __uint_as_float((unsigned)w);
  unsigned long long t0 = 0, t = 0;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t0));
  unsigned ns = 32;
  for (;;) {
    __nanosleep(ns);
    if (ns < 256) ns *= 2;
    w = ld_relaxed_gpu_u64(p);
    if ((unsigned)(w >> 32) != 0u) return __uint_as_float((unsigned)w);
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    if (t - t0 > 4000000000ull) return __int_as_float(0x7fc00000);
  }
}

// Poll *p until its epoch half equals ep (the word lands in `w`); false after
// ~limit_ns.  The first `spins` polls do not sleep (a peer that is about to
// arrive costs one round trip, not a scheduler wake-up).
__device__ __forceinline__ bool wait_word(const u64* p, unsigned ep, u64& w, unsigned long long limit_ns,
                                          int spins) {
  for (int k = 0; k < spins; ++k) {
    w = ld_relaxed_sys_u64(p);
    if ((unsigned)(w >> 32) == ep) return true;
  }
  unsigned long long t0 = 0;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t0));
  unsigned ns = 32;
  for (;;) {
    w = ld_relaxed_sys_u64(p);
    if ((unsigned)(w >> 32) == ep) return true;
    unsigned long long t = 0;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    if (t - t0 > limit_ns) return false;
    __nanosleep(ns);
    if (ns < 256) ns *= 2;
  }
}

}  // namespace fop

struct FopArgs {
  char* p[16];
  char* ws;
  char* peer[8];     // exchange buffers of the peer group as seen from this GPU (fop_peer_group)
  unsigned rank;     // this GPU's index in the peer group
  unsigned world;
  unsigned zero;     // always 0: the opaque zero of fop::nofuse (the runtime zero-fills FopArgs)
};
