// vs_score.cu -- the scoring kernel: pose transform + pairwise energy + per-pose reduction.
//
// score(pose) = sum_i sum_j e(i, j)   (pair terms DESIGN.md R1-R8)
//
// Layout of one CTA:
//   lane  = one pose of a 32-pose block of one spot;
//   warp  = one group of K_SLOTS ligand atoms (transformed coordinates and the
//           per-atom accumulators Q, A, B, H6, H5 live in registers);
//   the spot's receptor list streams through a NSTAGE-deep shared-memory ring
//   filled by the bulk-copy (TMA) engine; every lane reads the same receptor
//   atom (warp-uniform broadcast LDS.128).
// Energy of slot i after the sweep over the list:
//   E_i = es_i Q_i + c12_i A_i - c6_i B_i + C H6_i - D H5_i
//   Q_i = sum_j q_j S(r2)/r2 (DDD) , A_i = sum_j c12_j / r^12, B_i = sum_j c6_j / r^6,
//   H6_i = sum_j w_ij / r^12, H5_i = sum_j w_ij / r^10.
// The per-pose sum over slots and warps is done in a fixed order
// (deterministic: identical poses give identical fp32 scores).
#include "vs_kernels.cuh"

namespace vsk {

__device__ __forceinline__ void locate(const ScoreArgs& a, int bx, int& k, int& blk) {
  if (a.uniform) {
    k = bx / a.bps;
    blk = bx - k * a.bps;
  } else {  // largest k with blk_prefix[k] <= bx
    int lo = 0, hi = a.nseg - 1;
    while (lo < hi) {
      int mid = (lo + hi + 1) >> 1;
      if (__ldg(a.blk_prefix + mid) <= bx) lo = mid; else hi = mid - 1;
    }
    k = lo;
    blk = bx - __ldg(a.blk_prefix + k);
  }
}

template <int MODE, bool CUT, int DIEL>
__global__ void __launch_bounds__(GROUPS_PER_CTA * 32, 2) score_kernel(const ScoreArgs a) {
  __shared__ __align__(128) RecAtom tile[NSTAGE][TILE];
  __shared__ __align__(8) uint64_t full[NSTAGE];
  __shared__ double red[GROUPS_PER_CTA][32];

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int nwarps = blockDim.x >> 5;
  const int chunk = blockIdx.y;
  if (!a.uniform && (int)blockIdx.x >= __ldg(a.blk_prefix + a.nseg)) return;  // grid is an upper bound
  int k, blk;
  locate(a, blockIdx.x, k, blk);
  const int seg_n = a.uniform ? a.seg_size : (__ldg(a.pose_prefix + k + 1) - __ldg(a.pose_prefix + k));
  const int p0 = blk * POSES_PER_CTA;
  const int cnt = min(POSES_PER_CTA, seg_n - p0);
  const int spot = __ldg(a.seg_spot + k);
  const bool active = lane < cnt;
  const int p = p0 + (active ? lane : 0);
  const int item = (a.uniform ? k * a.seg_size : __ldg(a.pose_prefix + k)) + p;

  // ---- pose of this lane (PLAIN: given; LS: proposal around X[j], R16)
  float4 q, t;
  int jx = 0, j = 0;
  float old_score = 0.0f;
  if (MODE == MODE_PLAIN) {
    const int pidx = a.uniform ? k * a.seg_stride + p : item;
    const PoseRec r = a.poses[pidx];
    q = r.q;
    t = r.t;
  } else {
    j = __ldg(a.J + k * a.m + p);
    jx = k * a.P + j;
    const PoseRec r = a.poses[jx];
    q = r.q;
    t = r.t;
    old_score = r.t.w;
    perturb(q, t, a.ls_trans, a.ls_rot, a.T, a.seed, (uint32_t)j, (uint32_t)spot, (uint32_t)a.g, TAG_LS,
            2u * (uint32_t)a.l);
  }

  // ---- rotation (homogeneous form, R11) and transformed ligand slots
  float X[K_SLOTS], Y[K_SLOTS], Z[K_SLOTS];
  float DN[K_SLOTS], AC[K_SLOTS];
  {
    const float w = q.x, x = q.y, y = q.z, z = q.w;
    const float s2 = 2.0f / (w * w + x * x + y * y + z * z);
    const float r00 = 1.0f - s2 * (y * y + z * z), r01 = s2 * (x * y - w * z), r02 = s2 * (x * z + w * y);
    const float r10 = s2 * (x * y + w * z), r11 = 1.0f - s2 * (x * x + z * z), r12 = s2 * (y * z - w * x);
    const float r20 = s2 * (x * z - w * y), r21 = s2 * (y * z + w * x), r22 = 1.0f - s2 * (x * x + y * y);
    const float4 sh = __ldg(a.shift + spot);
    const float ox = sh.x + t.x, oy = sh.y + t.y, oz = sh.z + t.z;
    const LigSlot* L = a.lig + (size_t)(chunk * GROUPS_PER_CTA + warp) * K_SLOTS;
#pragma unroll
    for (int s = 0; s < K_SLOTS; ++s) {
      const float4 l = __ldg(&L[s].lq);
      const float4 pp = __ldg(&L[s].p);
      X[s] = ox + (r00 * l.x + r01 * l.y + r02 * l.z);
      Y[s] = oy + (r10 * l.x + r11 * l.y + r12 * l.z);
      Z[s] = oz + (r20 * l.x + r21 * l.y + r22 * l.z);
      DN[s] = pp.z;
      AC[s] = pp.w;
    }
  }
  float Q[K_SLOTS], A[K_SLOTS], B[K_SLOTS], H6[K_SLOTS], H5[K_SLOTS];
#pragma unroll
  for (int s = 0; s < K_SLOTS; ++s) Q[s] = A[s] = B[s] = H6[s] = H5[s] = 0.0f;

  // ---- receptor list of the spot through the bulk-copy ring
  const int off = __ldg(a.list_off + spot), len = __ldg(a.list_len + spot);
  const RecAtom* src = a.lists + off;
  const int nt = (len + TILE - 1) / TILE;
  if (threadIdx.x == 0) {
    for (int s = 0; s < NSTAGE; ++s) mbar_init(&full[s], 1);
    fence_mbar_init();
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    for (int s = 0; s < NSTAGE && s < nt; ++s) {
      const uint32_t bytes = (uint32_t)min(TILE, len - s * TILE) * (uint32_t)sizeof(RecAtom);
      mbar_arrive_expect_tx(&full[s], bytes);
      bulk_g2s(tile[s], src + (size_t)s * TILE, bytes, &full[s]);
    }
  }
  const float r2min = a.r2min, rc2 = a.rc2, inv_rc2 = a.inv_rc2;
  for (int it = 0; it < nt; ++it) {
    const int st = it % NSTAGE;
    mbar_wait(&full[st], (uint32_t)(it / NSTAGE) & 1u);
    const int nvalid = min(TILE, len - it * TILE);
    const RecAtom* T = tile[st];
#pragma unroll 1
    for (int r = 0; r < nvalid; ++r) {
      const float4 xq = T[r].xq;
      const float4 pp = T[r].p;
#pragma unroll
      for (int s = 0; s < K_SLOTS; ++s) {
        const float dx = X[s] - xq.x, dy = Y[s] - xq.y, dz = Z[s] - xq.z;
        float r2 = fmaf(dx, dx, fmaf(dy, dy, dz * dz));
        r2 = fmaxf(r2, r2min);                                   // R7
        float sh = 1.0f;
        if (CUT) {
          sh = fmaf(r2, -inv_rc2, 1.0f);                         // 1 - r2/rc2 (R6)
          r2 = (r2 < rc2) ? r2 : __int_as_float(0x7f800000);     // beyond rc: 1/r2 -> 0
        }
        const float inv = rcp_approx(r2);
        float es = (DIEL == 0) ? inv : rsqrt_approx(r2);
        if (CUT) es = (es * sh) * sh;
        Q[s] = fmaf(xq.w, es, Q[s]);
        const float inv2 = inv * inv, inv3 = inv2 * inv, inv6 = inv3 * inv3, inv5 = inv3 * inv2;
        A[s] = fmaf(pp.x, inv6, A[s]);
        B[s] = fmaf(pp.y, inv3, B[s]);
        const float w = fmaf(DN[s], pp.w, AC[s] * pp.z);           // donor_i acc_j + acc_i donor_j (R5)
        H6[s] = fmaf(w, inv6, H6[s]);
        H5[s] = fmaf(w, inv5, H5[s]);
      }
    }
    __syncthreads();  // every warp is done with stage st
    if (threadIdx.x == 0 && it + NSTAGE < nt) {
      const int nx = it + NSTAGE;
      const uint32_t bytes = (uint32_t)min(TILE, len - nx * TILE) * (uint32_t)sizeof(RecAtom);
      mbar_arrive_expect_tx(&full[st], bytes);
      bulk_g2s(tile[st], src + (size_t)nx * TILE, bytes, &full[st]);
    }
  }

  // ---- per-slot energies (fp64 combination of the fp32 sums: the terms cancel), fixed-order reduction
  double e = 0.0;
  {
    const LigSlot* L = a.lig + (size_t)(chunk * GROUPS_PER_CTA + warp) * K_SLOTS;
#pragma unroll
    for (int s = 0; s < K_SLOTS; ++s) {
      const float4 l = __ldg(&L[s].lq);
      const float4 pp = __ldg(&L[s].p);
      double es = (double)l.w * (double)Q[s];
      es = fma((double)pp.x, (double)A[s], es);
      es = fma(-(double)pp.y, (double)B[s], es);
      es = fma((double)a.hbC, (double)H6[s], es);
      es = fma(-(double)a.hbD, (double)H5[s], es);
      e += es;
    }
  }
  red[warp][lane] = e;
  __syncthreads();
  if (warp == 0) {
    double sum = 0.0;
    for (int w = 0; w < nwarps; ++w) sum += red[w][lane];
    const float score = (float)sum;
    if (active) {
      if (a.n_chunks > 1) {
        a.partial[(size_t)item * a.n_chunks + chunk] = sum;
      } else if (MODE == MODE_PLAIN) {
        const int pidx = a.uniform ? k * a.seg_stride + p : item;
        a.poses[pidx].t.w = score;
        if (a.orig) a.score_out[__ldg(a.orig + pidx)] = score;
      } else if (score < old_score) {                            // strict improvement (R16)
        PoseRec r;
        r.q = q;
        r.t = make_float4(t.x, t.y, t.z, score);
        a.poses[jx] = r;
      }
    }
    if (lane == 0 && chunk == 0 && a.counters) {
      atomicAdd(a.counters + 0, (unsigned long long)cnt * (unsigned long long)a.n_lig * (unsigned long long)len);
      atomicAdd(a.counters + 1, (unsigned long long)cnt);
    }
  }
}

// multi-chunk ligands: fixed-order sum of the chunk partials + the epilogue
template <int MODE>
__global__ void finalize_kernel(const ScoreArgs a, int n_items_blocks) {
  const int bx = blockIdx.x;
  if (bx >= n_items_blocks) return;
  if (!a.uniform && bx >= __ldg(a.blk_prefix + a.nseg)) return;
  int k, blk;
  locate(a, bx, k, blk);
  const int seg_n = a.uniform ? a.seg_size : (__ldg(a.pose_prefix + k + 1) - __ldg(a.pose_prefix + k));
  const int p = blk * POSES_PER_CTA + threadIdx.x;
  if (p >= seg_n) return;
  const int item = (a.uniform ? k * a.seg_size : __ldg(a.pose_prefix + k)) + p;
  double sum = 0.0;
  for (int c = 0; c < a.n_chunks; ++c) sum += a.partial[(size_t)item * a.n_chunks + c];
  const float score = (float)sum;
  if (MODE == MODE_PLAIN) {
    const int pidx = a.uniform ? k * a.seg_stride + p : item;
    a.poses[pidx].t.w = score;
    if (a.orig) a.score_out[__ldg(a.orig + pidx)] = score;
  } else {
    const int spot = __ldg(a.seg_spot + k);
    const int j = __ldg(a.J + k * a.m + p);
    const int jx = k * a.P + j;
    PoseRec r = a.poses[jx];
    if (score < r.t.w) {
      float4 q = r.q, t = r.t;
      perturb(q, t, a.ls_trans, a.ls_rot, a.T, a.seed, (uint32_t)j, (uint32_t)spot, (uint32_t)a.g, TAG_LS,
              2u * (uint32_t)a.l);
      r.q = q;
      r.t = make_float4(t.x, t.y, t.z, score);
      a.poses[jx] = r;
    }
  }
}

template <int MODE, bool CUT>
static cudaError_t launch_diel(const ScoreArgs& a, int diel, dim3 grid, dim3 block, cudaStream_t st) {
  if (diel == 0)
    score_kernel<MODE, CUT, 0><<<grid, block, 0, st>>>(a);
  else
    score_kernel<MODE, CUT, 1><<<grid, block, 0, st>>>(a);
  return cudaGetLastError();
}

cudaError_t launch_score(const ScoreArgs& a, int mode, bool cutoff, int dielectric, int n_blocks, cudaStream_t st) {
  if (n_blocks <= 0) return cudaSuccess;
  const int warps = a.n_chunks > 1 ? GROUPS_PER_CTA : a.n_groups;
  dim3 grid(n_blocks, a.n_chunks), block(warps * 32);
  if (mode == MODE_PLAIN)
    return cutoff ? launch_diel<MODE_PLAIN, true>(a, dielectric, grid, block, st)
                  : launch_diel<MODE_PLAIN, false>(a, dielectric, grid, block, st);
  return cutoff ? launch_diel<MODE_LS, true>(a, dielectric, grid, block, st)
                : launch_diel<MODE_LS, false>(a, dielectric, grid, block, st);
}

cudaError_t launch_finalize(const ScoreArgs& a, int mode, int n_blocks, cudaStream_t st) {
  if (n_blocks <= 0) return cudaSuccess;
  if (mode == MODE_PLAIN)
    finalize_kernel<MODE_PLAIN><<<n_blocks, POSES_PER_CTA, 0, st>>>(a, n_blocks);
  else
    finalize_kernel<MODE_LS><<<n_blocks, POSES_PER_CTA, 0, st>>>(a, n_blocks);
  return cudaGetLastError();
}

}  // namespace vsk
