// vs_pop.cu -- population kernels of Algorithm 1 + list building.
//
//   init_kernel      Initialize(S): uniform random rotation + translation (R12)
//   combine_kernel   Select + Combine: rank tournaments, blend crossover, mutation (R13-R15)
//   popsort_kernel   (score, index) bitonic sort per spot: Improve's choice of the
//                    best m (R17), the generation-0 sort, Include (R19)
//   best_kernel      S[0] of every spot
//   list_kernel      per-spot receptor lists within reach (R10), order-preserving
// All pose arithmetic is single IEEE fp32 ops (R24) so the streams are
// byte-identical to any other implementation of the same reading.
#include "vs_kernels.cuh"

namespace vsk {

__global__ void init_kernel(PoseRec* S, int n_sel, int P, const int* seg_spot, const uint64_t* seedp, float T, int trig) {
  pdl_enter(trig);  // PDL: predecessor complete and visible (vs_kernels.cuh)
  const uint64_t seed = *seedp;
  const int idx = blockIdx.x * blockDim.x + threadIdx.x;
  if (idx >= n_sel * P) return;
  const int k = idx / P, i = idx - k * P;
  const uint32_t s = (uint32_t)__ldg(seg_spot + k);
  PoseRec r;
  r.q = rand_quat(seed, (uint32_t)i, s, 0u);
  const uint4 w = stream(seed, (uint32_t)i, s, 0u, TAG_INIT_TRANS, 0u);
  r.t = make_float4(__fmul_rn(T, v11(w.x)), __fmul_rn(T, v11(w.y)), __fmul_rn(T, v11(w.z)), 0.0f);
  S[idx] = r;
}

// child j of generation g from the sorted population S (rank = index)
__global__ void combine_kernel(const PoseRec* __restrict__ S, PoseRec* __restrict__ C, int n_sel, int P,
                               const int* seg_spot, const uint64_t* seedp, int g, float p_mut, float mut_trans,
                               float mut_rot, float T, int trig) {
  pdl_enter(trig);  // PDL: predecessor complete and visible (vs_kernels.cuh)
  const uint64_t seed = *seedp;
  const int idx = blockIdx.x * blockDim.x + threadIdx.x;
  if (idx >= n_sel * P) return;
  const int k = idx / P, j = idx - k * P;
  const uint32_t s = (uint32_t)__ldg(seg_spot + k);
  const uint32_t uP = (uint32_t)P;
  // Select: two binary tournaments on ranks (R13)
  const uint4 w = stream(seed, (uint32_t)j, s, (uint32_t)g, TAG_PARENT, 0u);
  const int p1 = (int)min(w.x % uP, w.y % uP);
  int p2 = (int)min(w.z % uP, w.w % uP);
  if (p2 == p1) p2 = (p1 + 1) % P;
  const PoseRec A = S[(size_t)k * P + p1];
  const PoseRec B = S[(size_t)k * P + p2];
  // Combine: blend crossover (R14)
  const float alpha = u01(stream(seed, (uint32_t)j, s, (uint32_t)g, TAG_CROSS, 0u).x);
  const float beta = __fsub_rn(1.0f, alpha);
  float4 t;
  t.x = __fadd_rn(A.t.x, __fmul_rn(alpha, __fsub_rn(B.t.x, A.t.x)));
  t.y = __fadd_rn(A.t.y, __fmul_rn(alpha, __fsub_rn(B.t.y, A.t.y)));
  t.z = __fadd_rn(A.t.z, __fmul_rn(alpha, __fsub_rn(B.t.z, A.t.z)));
  t.w = 0.0f;
  const float dot = __fadd_rn(__fadd_rn(__fadd_rn(__fmul_rn(A.q.x, B.q.x), __fmul_rn(A.q.y, B.q.y)),
                                        __fmul_rn(A.q.z, B.q.z)), __fmul_rn(A.q.w, B.q.w));
  float4 q2 = B.q;
  if (dot < 0.0f) q2 = make_float4(-q2.x, -q2.y, -q2.z, -q2.w);
  float4 q = make_float4(__fadd_rn(__fmul_rn(beta, A.q.x), __fmul_rn(alpha, q2.x)),
                         __fadd_rn(__fmul_rn(beta, A.q.y), __fmul_rn(alpha, q2.y)),
                         __fadd_rn(__fmul_rn(beta, A.q.z), __fmul_rn(alpha, q2.z)),
                         __fadd_rn(__fmul_rn(beta, A.q.w), __fmul_rn(alpha, q2.w)));
  q = normalize_q(q);
  // mutation (R15)
  if (u01(stream(seed, (uint32_t)j, s, (uint32_t)g, TAG_MUT, 0u).x) < p_mut)
    perturb(q, t, mut_trans, mut_rot, T, seed, (uint32_t)j, s, (uint32_t)g, TAG_MUT, 1u);
  PoseRec r;
  r.q = q;
  r.t = t;
  C[idx] = r;
}

__device__ __forceinline__ uint64_t pkey(float score, uint32_t idx) {
  return ((uint64_t)ord_f32(score) << 32) | idx;
}

// One CTA per spot.  mode 0: J = best m of S by (score, index);
// mode 1: S_out = S sorted; mode 2: S_out = best P of S ++ C (S first on ties).
__global__ void popsort_kernel(int mode, const PoseRec* __restrict__ S, const PoseRec* __restrict__ C,
                               PoseRec* __restrict__ S_out, int* __restrict__ J, int P, int m, int N, int trig) {
  pdl_enter(trig);  // PDL: predecessor complete and visible (vs_kernels.cuh)
  extern __shared__ uint64_t keys[];
  const int k = blockIdx.x;
  const int count = mode == 2 ? 2 * P : P;
  const PoseRec* Sk = S + (size_t)k * P;
  const PoseRec* Ck = C ? C + (size_t)k * P : nullptr;
  for (int i = threadIdx.x; i < N; i += blockDim.x) {
    uint64_t key = ~0ull;
    if (i < P) key = pkey(Sk[i].t.w, (uint32_t)i);
    else if (i < count) key = pkey(Ck[i - P].t.w, (uint32_t)i);
    keys[i] = key;
  }
  __syncthreads();
  for (int size = 2; size <= N; size <<= 1) {
    for (int stride = size >> 1; stride > 0; stride >>= 1) {
      for (int i = threadIdx.x; i < (N >> 1); i += blockDim.x) {
        const int lo = 2 * i - (i & (stride - 1));
        const int hi = lo + stride;
        const bool asc = (lo & size) == 0;
        const uint64_t a = keys[lo], b = keys[hi];
        if ((a > b) == asc) {
          keys[lo] = b;
          keys[hi] = a;
        }
      }
      __syncthreads();
    }
  }
  if (mode == 0) {  // the best m by (score, index), in that order
    for (int r = threadIdx.x; r < m; r += blockDim.x) J[(size_t)k * m + r] = (int)(uint32_t)keys[r];
  } else {
    for (int r = threadIdx.x; r < P; r += blockDim.x) {
      const int o = (int)(uint32_t)keys[r];
      S_out[(size_t)k * P + r] = o < P ? Sk[o] : Ck[o - P];
    }
  }
}

__global__ void best_kernel(const PoseRec* S, int n_sel, int P, float* best_pose, float* best_score) {
  pdl_enter();  // PDL: predecessor complete and visible (vs_kernels.cuh)
  const int k = blockIdx.x * blockDim.x + threadIdx.x;
  if (k >= n_sel) return;
  const PoseRec r = S[(size_t)k * P];
  float* o = best_pose + 7 * (size_t)k;
  o[0] = r.q.x; o[1] = r.q.y; o[2] = r.q.z; o[3] = r.q.w;
  o[4] = r.t.x; o[5] = r.t.y; o[6] = r.t.z;
  best_score[k] = r.t.w;
}

// Per-spot receptor list: atoms with |r_j - c_s|^2 <= reach2 in receptor order,
// stored relative to c_s.  One CTA per spot; count pass then fill pass.
__global__ void list_kernel(const float4* __restrict__ rec, const float4* __restrict__ rprm, int n_rec,
                            const float4* __restrict__ spot_c, float reach2, const int* __restrict__ off,
                            int* __restrict__ len, RecAtom* __restrict__ lists, int count_only) {
  __shared__ int warp_cnt[32];
  __shared__ int base_sh;
  const int s = blockIdx.x;
  const float4 c = spot_c[s];
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, nw = blockDim.x >> 5;
  if (threadIdx.x == 0) base_sh = 0;
  __syncthreads();
  RecAtom* out = count_only ? nullptr : lists + off[s];
  for (int b = 0; b < n_rec; b += blockDim.x) {
    const int j = b + threadIdx.x;
    bool in = false;
    float4 x = make_float4(0, 0, 0, 0);
    if (j < n_rec) {
      x = rec[j];
      const float dx = __fsub_rn(x.x, c.x), dy = __fsub_rn(x.y, c.y), dz = __fsub_rn(x.z, c.z);
      x.x = dx; x.y = dy; x.z = dz;
      in = (dx * dx + dy * dy + dz * dz) <= reach2;
    }
    const unsigned ball = __ballot_sync(0xffffffffu, in);
    if (lane == 0) warp_cnt[warp] = __popc(ball);
    __syncthreads();
    int before = 0, total = 0;
    for (int w = 0; w < nw; ++w) {
      const int cw = warp_cnt[w];
      if (w < warp) before += cw;
      total += cw;
    }
    const int pos = base_sh + before + __popc(ball & ((1u << lane) - 1u));
    if (in && out) {
      RecAtom a;
      a.xq = x;
      a.p = rprm[j];
      out[pos] = a;
    }
    __syncthreads();
    if (threadIdx.x == 0) base_sh += total;
    __syncthreads();
  }
  if (threadIdx.x == 0 && count_only) len[s] = base_sh;
}

__global__ void philox_kernel(int64_t n, const uint4* ctr, uint2 key, uint4* out) {
  const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i < n) out[i] = philox4x32_10(ctr[i], key);
}

// vs_score_poses_device: validation + per-spot counts
__global__ void validate_kernel(int64_t n, const int32_t* spot, const float* q, const float* t, int n_spots, float T,
                                int cutoff, int* valid, int* counts, float* score_out) {
  const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  const int s = spot[i];
  bool ok = s >= 0 && s < n_spots;
  float qq[4], tt[3];
  bool nz = false;
  for (int c = 0; c < 4; ++c) { qq[c] = q[4 * i + c]; ok = ok && isfinite(qq[c]); nz = nz || qq[c] != 0.0f; }
  for (int c = 0; c < 3; ++c) {
    tt[c] = t[3 * i + c];
    ok = ok && isfinite(tt[c]);
    if (cutoff) ok = ok && fabsf(tt[c]) <= T;
  }
  ok = ok && nz;
  valid[i] = ok ? 1 : 0;
  if (ok) atomicAdd(counts + s, 1);
  else score_out[i] = __int_as_float(0x7fc00000);
}

__global__ void scatter_kernel(int64_t n, const int32_t* spot, const float* q, const float* t, const int* valid,
                               int* cursor, PoseRec* sorted, int* orig) {
  const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n || !valid[i]) return;
  const int pos = atomicAdd(cursor + spot[i], 1);
  PoseRec r;
  r.q = make_float4(q[4 * i], q[4 * i + 1], q[4 * i + 2], q[4 * i + 3]);
  r.t = make_float4(t[3 * i], t[3 * i + 1], t[3 * i + 2], 0.0f);
  sorted[pos] = r;
  orig[pos] = (int)i;
}

// ---------------------------------------------------------------- launchers
static inline int nblk(int64_t n, int b) { return (int)((n + b - 1) / b); }

cudaError_t launch_init(PoseRec* S, int n_sel, int P, const int* seg_spot, const uint64_t* seedp, float T, int trig,
                        cudaStream_t st) {
  return launch_chain(init_kernel, nblk((int64_t)n_sel * P, 128), 128, 0, st, S, n_sel, P, seg_spot, seedp, T, trig);
}

cudaError_t launch_combine(const PoseRec* S, PoseRec* C, int n_sel, int P, const int* seg_spot, const uint64_t* seedp, int g,
                           float p_mut, float mut_trans, float mut_rot, float T, int trig, cudaStream_t st) {
  return launch_chain(combine_kernel, nblk((int64_t)n_sel * P, 128), 128, 0, st, S, C, n_sel, P, seg_spot, seedp, g, p_mut,
                      mut_trans, mut_rot, T, trig);
}

cudaError_t launch_popsort(int mode, const PoseRec* S, const PoseRec* C, PoseRec* S_out, int* J, int n_sel, int P,
                           int m, int trig, cudaStream_t st) {
  const int count = mode == 2 ? 2 * P : P;
  int N = 2;
  while (N < count) N <<= 1;
  const int threads = min(1024, max(32, N / 2));
  const size_t smem = sizeof(uint64_t) * N;
  return launch_chain(popsort_kernel, n_sel, threads, smem, st, mode, S, C, S_out, J, P, m, N, trig);
}

cudaError_t launch_best(const PoseRec* S, int n_sel, int P, float* best_pose, float* best_score, cudaStream_t st) {
  return launch_chain(best_kernel, nblk(n_sel, 128), 128, 0, st, S, n_sel, P, best_pose, best_score);
}

cudaError_t launch_build_lists(const float4* rec, const float4* rprm, int n_rec, const float4* spot_c, int n_spots,
                               float reach2, const int* off, int* len, RecAtom* lists, int count_only,
                               cudaStream_t st) {
  list_kernel<<<n_spots, 256, 0, st>>>(rec, rprm, n_rec, spot_c, reach2, off, len, lists, count_only);
  return cudaGetLastError();
}

cudaError_t launch_philox(int64_t n, const uint4* ctr, uint2 key, uint4* out, cudaStream_t st) {
  if (n <= 0) return cudaSuccess;
  philox_kernel<<<nblk(n, 256), 256, 0, st>>>(n, ctr, key, out);
  return cudaGetLastError();
}

cudaError_t launch_validate(int64_t n, const int32_t* spot, const float* q, const float* t, int n_spots, float T,
                            int cutoff, int* valid, int* counts, float* score_out, cudaStream_t st) {
  validate_kernel<<<nblk(n, 256), 256, 0, st>>>(n, spot, q, t, n_spots, T, cutoff, valid, counts, score_out);
  return cudaGetLastError();
}

cudaError_t launch_scatter(int64_t n, const int32_t* spot, const float* q, const float* t, const int* valid,
                           int* cursor, PoseRec* sorted, int* orig, cudaStream_t st) {
  scatter_kernel<<<nblk(n, 256), 256, 0, st>>>(n, spot, q, t, valid, cursor, sorted, orig);
  return cudaGetLastError();
}

}  // namespace vsk
