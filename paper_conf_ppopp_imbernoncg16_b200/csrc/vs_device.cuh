// vs_device.cuh -- device-side building blocks of the B200 hot path.
//
// Philox4x32-10 streams (R23), the fp32 pose operators of the
// metaheuristic written as single IEEE ops (R24: __f*_rn intrinsics are
// never contracted into FMA), and the cp.async primitives used to stage
// receptor atoms in shared memory ("tiling via shared
// memory").  Independent of oracle/ (shares no code with it).
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

namespace vsk {

// ---------------------------------------------------------------- records
// Receptor atom as streamed by the pair kernel: 32 B, two float4 so one
// warp-uniform LDS.128 pair broadcasts it to every lane.
struct __align__(16) RecAtom {
  float4 xq;  // x, y, z relative to the list origin (A), charge q_j (e)
  float4 p;   // c12_j, c6_j, donor_j (0/1), acceptor_j (0/1)
};

// Individual of a population: 32 B.
struct __align__(16) PoseRec {
  float4 q;   // w, x, y, z
  float4 t;   // tx, ty, tz, score
};

enum : uint32_t { TAG_INIT_ROT = 1, TAG_INIT_TRANS = 2, TAG_PARENT = 3, TAG_CROSS = 4, TAG_MUT = 5, TAG_LS = 6 };

// ---------------------------------------------------------------- Philox
__device__ __forceinline__ uint4 philox4x32_10(uint4 c, uint2 k) {
  const uint32_t M0 = 0xD2511F53u, M1 = 0xCD9E8D57u, W0 = 0x9E3779B9u, W1 = 0xBB67AE85u;
#pragma unroll
  for (int r = 0; r < 10; ++r) {
    if (r > 0) { k.x += W0; k.y += W1; }
    const uint32_t hi0 = __umulhi(M0, c.x), lo0 = M0 * c.x;
    const uint32_t hi1 = __umulhi(M1, c.z), lo1 = M1 * c.z;
    c = make_uint4(hi1 ^ c.y ^ k.x, lo1, hi0 ^ c.w ^ k.y, lo0);
  }
  return c;
}

// stream(i, s, g, tag, k): counter (i, s, g, tag<<24 | k), key = seed halves (R23)
__device__ __forceinline__ uint4 stream(uint64_t seed, uint32_t i, uint32_t s, uint32_t g, uint32_t tag, uint32_t k) {
  return philox4x32_10(make_uint4(i, s, g, (tag << 24) | k), make_uint2((uint32_t)seed, (uint32_t)(seed >> 32)));
}

__device__ __forceinline__ float u01(uint32_t w) { return __fmul_rn(__uint2float_rn(w >> 8), 5.9604644775390625e-08f); }
__device__ __forceinline__ float v11(uint32_t w) { return __fsub_rn(__fmul_rn(2.0f, u01(w)), 1.0f); }

// ---------------------------------------------------------------- fp32 pose operators (R24)
__device__ __forceinline__ float4 normalize_q(float4 q) {
  float n2 = __fadd_rn(__fadd_rn(__fadd_rn(__fmul_rn(q.x, q.x), __fmul_rn(q.y, q.y)), __fmul_rn(q.z, q.z)),
                       __fmul_rn(q.w, q.w));
  float n = __fsqrt_rn(n2);
  return make_float4(__fdiv_rn(q.x, n), __fdiv_rn(q.y, n), __fdiv_rn(q.z, n), __fdiv_rn(q.w, n));
}

// Hamilton product a (x) b; float4 = (w, x, y, z) in (.x, .y, .z, .w)
__device__ __forceinline__ float4 hamilton(float4 a, float4 b) {
  float w = __fsub_rn(__fsub_rn(__fsub_rn(__fmul_rn(a.x, b.x), __fmul_rn(a.y, b.y)), __fmul_rn(a.z, b.z)), __fmul_rn(a.w, b.w));
  float x = __fsub_rn(__fadd_rn(__fadd_rn(__fmul_rn(a.x, b.y), __fmul_rn(a.y, b.x)), __fmul_rn(a.z, b.w)), __fmul_rn(a.w, b.z));
  float y = __fadd_rn(__fadd_rn(__fsub_rn(__fmul_rn(a.x, b.z), __fmul_rn(a.y, b.w)), __fmul_rn(a.z, b.x)), __fmul_rn(a.w, b.y));
  float z = __fadd_rn(__fsub_rn(__fadd_rn(__fmul_rn(a.x, b.w), __fmul_rn(a.y, b.z)), __fmul_rn(a.z, b.y)), __fmul_rn(a.w, b.x));
  return make_float4(w, x, y, z);
}

// uniform rotation by rejection in the 4-ball (R12)
__device__ __forceinline__ float4 rand_quat(uint64_t seed, uint32_t i, uint32_t s, uint32_t g) {
  for (uint32_t k = 0; k < 64; ++k) {
    uint4 w = stream(seed, i, s, g, TAG_INIT_ROT, k);
    float a = v11(w.x), b = v11(w.y), c = v11(w.z), d = v11(w.w);
    float n2 = __fadd_rn(__fadd_rn(__fadd_rn(__fmul_rn(a, a), __fmul_rn(b, b)), __fmul_rn(c, c)), __fmul_rn(d, d));
    if (n2 > 0.0f && n2 <= 1.0f) {
      float n = __fsqrt_rn(n2);
      return make_float4(__fdiv_rn(a, n), __fdiv_rn(b, n), __fdiv_rn(c, n), __fdiv_rn(d, n));
    }
  }
  return make_float4(1.0f, 0.0f, 0.0f, 0.0f);
}

__device__ __forceinline__ float clampT(float v, float T) { return fminf(fmaxf(v, -T), T); }

// move + rotate in the neighbourhood of a conformation (R16)
__device__ __forceinline__ void perturb(float4& q, float4& t, float dt, float dr, float T, uint64_t seed, uint32_t i,
                                        uint32_t s, uint32_t g, uint32_t tag, uint32_t k) {
  uint4 a = stream(seed, i, s, g, tag, k);
  uint4 b = stream(seed, i, s, g, tag, k + 1);
  t.x = clampT(__fadd_rn(t.x, __fmul_rn(dt, v11(a.x))), T);
  t.y = clampT(__fadd_rn(t.y, __fmul_rn(dt, v11(a.y))), T);
  t.z = clampT(__fadd_rn(t.z, __fmul_rn(dt, v11(a.z))), T);
  float4 dq = make_float4(1.0f, __fmul_rn(dr, v11(b.x)), __fmul_rn(dr, v11(b.y)), __fmul_rn(dr, v11(b.z)));
  q = normalize_q(hamilton(dq, q));
}

// ---------------------------------------------------------------- asynchronous copies
__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

// per-thread asynchronous 16-byte copy global -> shared (L2 only), grouped by commit / wait
__device__ __forceinline__ void cp_async16(void* dst, const void* src) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(smem_u32(dst)), "l"(src) : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void cp_async_wait() { asm volatile("cp.async.wait_group %0;" ::"n"(N) : "memory"); }

__device__ __forceinline__ float rcp_approx(float x) {
  float r;
  asm("rcp.approx.ftz.f32 %0, %1;" : "=f"(r) : "f"(x));
  return r;
}
__device__ __forceinline__ float rsqrt_approx(float x) {
  float r;
  asm("rsqrt.approx.ftz.f32 %0, %1;" : "=f"(r) : "f"(x));
  return r;
}

// total order on fp32 scores as uint32 (-0 == +0), for (score, index) sort keys
__device__ __forceinline__ uint32_t ord_f32(float f) {
  uint32_t b = __float_as_uint(f == 0.0f ? 0.0f : f);
  return (b & 0x80000000u) ? ~b : (b | 0x80000000u);
}

}  // namespace vsk
