// vs_score.cu -- the scoring kernel: pose transform + pairwise energy + per-pose reduction.
//
// score(pose) = sum_i sum_j e(i, j)   (pair terms DESIGN.md R1-R8)
//
// Layout of one CTA:
//   lane  = one pose of a 32-pose block of one spot;
//   warp  = one group of K_SLOTS ligand atoms, held as K_PAIRS float2 slot
//           pairs: transformed coordinates and the per-atom accumulators live
//           in registers and every fp32 add/mul/fma of the pair loop is a
//           packed FADD2/FMUL2/FFMA2 over two ligand atoms, with the receptor
//           atom's value as the broadcast operand;
//   the spot's receptor list streams through a NSTAGE-deep shared-memory ring
//   filled by the bulk-copy (TMA) engine; every lane reads the same receptor
//   atom (warp-uniform broadcast LDS.128).
// Ligand atoms are ordered on the host so that hydrogen-bond-capable atoms
// (donor HD, acceptor N/O; R5) come last: a group's first K_PAIRS - H pairs
// skip the H-bond arithmetic, and H (warp-uniform) selects a specialised loop.
// Energy of slot i after the sweep over the list:
//   E_i = es_i Q_i + c12_i A_i - c6_i B_i + C H6_i - D H5_i
//   Q_i = sum_j q_j S(r2)/r2 (DDD), A_i = sum_j c12_j / r^12, B_i = sum_j c6_j / r^6,
//   H6_i = sum_j w_ij / r^12, H5_i = sum_j w_ij / r^10.
// The per-slot combination and the per-pose sum over slots and warps run in
// fp64 in a fixed order (deterministic: identical poses -> identical scores).
#include "vs_kernels.cuh"

#ifndef VS_UNROLL
#define VS_UNROLL 4
#endif
#ifndef VS_MINB
#define VS_MINB (16 / GROUPS_PER_CTA)
#endif
#ifdef VS_MAXNREG
#define VS_REGCAP __maxnreg__(VS_MAXNREG)
#else
#define VS_REGCAP __launch_bounds__(GROUPS_PER_CTA * 32, VS_MINB)
#endif
#define VS_STR2(x) #x
#define VS_STR(x) VS_STR2(x)

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

__device__ __forceinline__ float2 f2(float v) { return make_float2(v, v); }

// The sweep of one warp over the spot's receptor list.  The group has H slot
// pairs with H-bond-capable atoms (warp-uniform, compile-time here): the first
// K_PAIRS - H pairs skip the H-bond arithmetic and keep no H-bond registers.
// Warps are decoupled: a warp releases a ring stage when it is done with it and
// the last warp to release a stage refills it (bulk copy), so a warp never
// waits for the others except on data that has not yet landed.
template <int H, bool CUT, int DIEL>
__device__ __forceinline__ double sweep(const ScoreArgs& a, const LigSlot* L, const float (&R)[9], float ox, float oy,
                                        float oz, RecAtom (*tile)[TILE], uint64_t* full, int* relcnt,
                                        const RecAtom* src, int len, int nt, int nwarps) {
  constexpr int HP = H > 0 ? H : 1;
  constexpr int P0 = K_PAIRS - H;  // first H-bond pair
  float2 X[K_PAIRS], Y[K_PAIRS], Z[K_PAIRS], Q[K_PAIRS], A[K_PAIRS], B[K_PAIRS];
  float2 H6[HP], H5[HP];
  bool DN[2 * HP];
#pragma unroll
  for (int p = 0; p < K_PAIRS; ++p) {
    const float4 l0 = __ldg(&L[2 * p].lq), l1 = __ldg(&L[2 * p + 1].lq);
    X[p] = make_float2(ox + (R[0] * l0.x + R[1] * l0.y + R[2] * l0.z), ox + (R[0] * l1.x + R[1] * l1.y + R[2] * l1.z));
    Y[p] = make_float2(oy + (R[3] * l0.x + R[4] * l0.y + R[5] * l0.z), oy + (R[3] * l1.x + R[4] * l1.y + R[5] * l1.z));
    Z[p] = make_float2(oz + (R[6] * l0.x + R[7] * l0.y + R[8] * l0.z), oz + (R[6] * l1.x + R[7] * l1.y + R[8] * l1.z));
    Q[p] = A[p] = B[p] = make_float2(0.0f, 0.0f);
    if (p >= P0) {
      H6[p - P0] = H5[p - P0] = make_float2(0.0f, 0.0f);
      DN[2 * (p - P0)] = __ldg(&L[2 * p].p.z) != 0.0f;
      DN[2 * (p - P0) + 1] = __ldg(&L[2 * p + 1].p.z) != 0.0f;
    }
  }
  const float r2min = a.r2min, rc2 = a.rc2, inv_rc2 = a.inv_rc2;
  const float INF = __int_as_float(0x7f800000);
  const int lane = threadIdx.x & 31;
  for (int it = 0; it < nt; ++it) {
    const int st = it % NSTAGE;
    mbar_wait(&full[st], (uint32_t)(it / NSTAGE) & 1u);
    const int nvalid = min(TILE, len - it * TILE);
    const RecAtom* T = tile[st];
    _Pragma(VS_STR(unroll VS_UNROLL))
    for (int j = 0; j < nvalid; ++j) {
      const float4 xq = T[j].xq;
      const float4 pp = T[j].p;
#pragma unroll
      for (int p = 0; p < K_PAIRS; ++p) {
        const float2 dx = __fadd2_rn(X[p], f2(-xq.x));
        const float2 dy = __fadd2_rn(Y[p], f2(-xq.y));
        const float2 dz = __fadd2_rn(Z[p], f2(-xq.z));
        float2 r2 = __fmul2_rn(dx, dx);
        r2 = __ffma2_rn(dy, dy, r2);
        r2 = __ffma2_rn(dz, dz, r2);
        r2.x = fmaxf(r2.x, r2min);                                   // R7
        r2.y = fmaxf(r2.y, r2min);
        bool inx = true, iny = true;
        const float2 r2u = r2;
        if (CUT) {
          inx = r2.x < rc2;
          iny = r2.y < rc2;
          r2.x = inx ? r2.x : INF;                                   // beyond rc: 1/r2 -> 0
          r2.y = iny ? r2.y : INF;
        }
        float2 inv;
        inv.x = rcp_approx(r2.x);
        inv.y = rcp_approx(r2.y);
        float2 es = inv;
        if (DIEL == 0) {
          // shifted DDD Coulomb (R6): S(r2)/r2 = (1 - r2/rc2)^2 / r2 = 1/r2 - 2/rc2 + r2/rc2^2
          if (CUT) {
            es = __fadd2_rn(__ffma2_rn(r2u, f2(inv_rc2 * inv_rc2), inv), f2(-2.0f * inv_rc2));
            es.x = inx ? es.x : 0.0f;
            es.y = iny ? es.y : 0.0f;
          }
        } else {
          es.x = rsqrt_approx(r2.x);
          es.y = rsqrt_approx(r2.y);
          if (CUT) {
            const float2 sh = __ffma2_rn(r2u, f2(-inv_rc2), f2(1.0f));   // 1 - r2/rc2
            es = __fmul2_rn(__fmul2_rn(es, sh), sh);
          }
        }
        Q[p] = __ffma2_rn(es, f2(xq.w), Q[p]);
        const float2 inv2 = __fmul2_rn(inv, inv);
        const float2 inv3 = __fmul2_rn(inv2, inv);
        const float2 inv6 = __fmul2_rn(inv3, inv3);
        A[p] = __ffma2_rn(inv6, f2(pp.x), A[p]);
        B[p] = __ffma2_rn(inv3, f2(pp.y), B[p]);
        if (p >= P0) {                                               // compile-time after unrolling
          const int hq = p - P0;
          const float2 inv5 = __fmul2_rn(inv3, inv2);
          // a donor slot bonds with receptor acceptors, an acceptor slot with receptor donors (R5)
          const float2 w = make_float2(DN[2 * hq] ? pp.w : pp.z, DN[2 * hq + 1] ? pp.w : pp.z);
          H6[hq] = __ffma2_rn(w, inv6, H6[hq]);
          H5[hq] = __ffma2_rn(w, inv5, H5[hq]);
        }
      }
    }
    // release stage st; the last warp to release it refills it with tile it + NSTAGE
    __syncwarp();
    if (lane == 0) {
      __threadfence_block();
      if (atomicAdd(&relcnt[st], 1) == nwarps - 1) {
        atomicExch(&relcnt[st], 0);
        if (it + NSTAGE < nt) {
          const int nx = it + NSTAGE;
          const uint32_t bytes = (uint32_t)min(TILE, len - nx * TILE) * (uint32_t)sizeof(RecAtom);
          fence_proxy_async();
          mbar_arrive_expect_tx(&full[st], bytes);
          bulk_g2s(tile[st], src + (size_t)nx * TILE, bytes, &full[st]);
        }
      }
    }
  }
  // per-slot energies: fp64 combination of the fp32 sums (the terms cancel)
  double e = 0.0;
#pragma unroll
  for (int s = 0; s < K_SLOTS; ++s) {
    const int p = s >> 1;
    const bool hi = s & 1;
    const float4 l = __ldg(&L[s].lq);
    const float4 pv = __ldg(&L[s].p);
    double es = (double)l.w * (double)(hi ? Q[p].y : Q[p].x);
    es = fma((double)pv.x, (double)(hi ? A[p].y : A[p].x), es);
    es = fma(-(double)pv.y, (double)(hi ? B[p].y : B[p].x), es);
    if (p >= P0) {
      const int hq = p - P0;
      const double hsel = (double)(pv.z + pv.w);  // 1 for donors / acceptors, 0 for padding atoms
      es = fma(hsel * a.hbC, (double)(hi ? H6[hq].y : H6[hq].x), es);
      es = fma(-hsel * a.hbD, (double)(hi ? H5[hq].y : H5[hq].x), es);
    }
    e += es;
  }
  return e;
}

template <int MODE, bool CUT, int DIEL>
__global__ void VS_REGCAP score_kernel(const ScoreArgs a) {
  __shared__ __align__(128) RecAtom tile[NSTAGE][TILE];
  __shared__ __align__(8) uint64_t full[NSTAGE];
  __shared__ int relcnt[NSTAGE];
  __shared__ double red[GROUPS_PER_CTA][32];

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int nwarps = blockDim.x >> 5;
  const int chunk = blockIdx.y;
  if (!a.uniform && (int)blockIdx.x >= __ldg(a.blk_prefix + a.nseg)) return;  // grid is an upper bound
  int k, blk;
  locate(a, blockIdx.x, k, blk);
  const int seg_n = a.uniform ? a.seg_size : (__ldg(a.pose_prefix + k + 1) - __ldg(a.pose_prefix + k));
  const int spot = __ldg(a.seg_spot + k);
  int cnt, p, group;
  if (a.mixed) {
    // lane -> (pose, ligand group) item of the segment, group-major: fills the lanes when the
    // segment has few poses (Improve's m = round(f P) poses per spot)
    const int n_items = seg_n * a.n_groups;
    const int it0 = blk * POSES_PER_CTA;
    cnt = min(POSES_PER_CTA, n_items - it0);
    const int itl = it0 + (lane < cnt ? lane : 0);
    group = itl / seg_n;
    p = itl - group * seg_n;
  } else {
    const int p0 = blk * POSES_PER_CTA;
    cnt = min(POSES_PER_CTA, seg_n - p0);
    p = p0 + (lane < cnt ? lane : 0);
    group = chunk * GROUPS_PER_CTA + warp;
  }
  const bool active = lane < cnt;
  const int item = (a.uniform ? k * a.seg_size : __ldg(a.pose_prefix + k)) + p;

  // ---- pose of this lane (PLAIN: given; LS: proposal around X[j], R16)
  float4 q, t;
  int jx = 0, j = 0;
  float old_score = 0.0f;
  if (MODE == MODE_PLAIN) {
    const int pidx = a.uniform ? k * a.seg_stride + (a.perm ? __ldg(a.perm + k * a.seg_size + p) : p) : item;
    const PoseRec r = a.poses[pidx];
    q = r.q;
    t = r.t;
  } else {
    const int jj = p / a.K, kk = p - jj * a.K;
    j = __ldg(a.J + k * a.m + jj);
    jx = k * a.P + j;
    const PoseRec r = a.poses[jx];
    q = r.q;
    t = r.t;
    old_score = r.t.w;
    perturb(q, t, a.ls_trans, a.ls_rot, a.T, *a.seedp, (uint32_t)j, (uint32_t)spot, (uint32_t)a.g, TAG_LS,
            2u * (uint32_t)(a.l * a.K + kk));
  }

  // ---- rotation (homogeneous form, R11)
  float R[9];
  float ox, oy, oz;
  {
    const float w = q.x, x = q.y, y = q.z, z = q.w;
    const float s2 = 2.0f / (w * w + x * x + y * y + z * z);
    R[0] = 1.0f - s2 * (y * y + z * z); R[1] = s2 * (x * y - w * z); R[2] = s2 * (x * z + w * y);
    R[3] = s2 * (x * y + w * z); R[4] = 1.0f - s2 * (x * x + z * z); R[5] = s2 * (y * z - w * x);
    R[6] = s2 * (x * z - w * y); R[7] = s2 * (y * z + w * x); R[8] = 1.0f - s2 * (x * x + y * y);
    const float4 sh = __ldg(a.shift + spot);
    ox = sh.x + t.x;
    oy = sh.y + t.y;
    oz = sh.z + t.z;
  }
  const LigSlot* L = a.lig + (size_t)group * K_SLOTS;

  // ---- receptor list of the spot through the bulk-copy ring
  const int off = __ldg(a.list_off + spot);
  int len = __ldg(a.list_len + spot);
  if (CUT && a.shell) {
    // the list is sorted by |r|: atoms farther than R_w + rc from the spot centre, R_w = max |x_i| over the
    // warp's ligand atoms, are beyond the cutoff of every pair of this warp -> stream only the inner shells
    float r2m = 0.0f;
#pragma unroll
    for (int sl = 0; sl < K_SLOTS; ++sl) {
      const float4 l = __ldg(&L[sl].lq);
      const float x = ox + (R[0] * l.x + R[1] * l.y + R[2] * l.z);
      const float y = oy + (R[3] * l.x + R[4] * l.y + R[5] * l.z);
      const float z = oz + (R[6] * l.x + R[7] * l.y + R[8] * l.z);
      r2m = fmaxf(r2m, x * x + y * y + z * z);
    }
    r2m = __uint_as_float(__reduce_max_sync(0xffffffffu, __float_as_uint(r2m)));
    const float reach = sqrtf(r2m) + a.rc + 0.01f;                 // 0.01 A absorbs fp32 rounding
    const int b = (int)ceilf(reach * (1.0f / SHELL_DR)) - 1;
    if (b < NSHELL) len = min(len, __ldg(a.shell + (size_t)spot * NSHELL + max(b, 0)));
  }
  // list split (launches too small to fill the GPU): this CTA streams tiles [t0, t1) of the list; the
  // split partial energies are summed in a fixed order by the CTA that completes the pose
  const int nt_all = (len + TILE - 1) / TILE;
  const int t0 = (int)(((long long)nt_all * blockIdx.z) / a.nsplit);
  const int t1 = (int)(((long long)nt_all * (blockIdx.z + 1)) / a.nsplit);
  const RecAtom* src = a.lists + off + (size_t)t0 * TILE;
  len = max(0, min(len, t1 * TILE) - t0 * TILE);
  const int nt = t1 - t0;
  if (threadIdx.x == 0) {
    for (int s = 0; s < NSTAGE; ++s) {
      mbar_init(&full[s], 1);
      relcnt[s] = 0;
    }
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
  // warp-uniform number of H-bond pairs in this warp's group (spread evenly over the groups); lanes of
  // mixed warps hold different groups and all run the largest count (the extra pairs carry zero weight)
  const int h = a.mixed ? a.hb_max : a.hb_base + (group < a.hb_extra ? 1 : 0);
  double e;
  switch (h) {
#define VS_CASE(HH) \
  case HH: e = sweep<(HH <= K_PAIRS ? HH : K_PAIRS), CUT, DIEL>(a, L, R, ox, oy, oz, tile, full, relcnt, src, len, nt, nwarps); break;
    VS_CASE(0) VS_CASE(1) VS_CASE(2) VS_CASE(3) VS_CASE(4) VS_CASE(5) VS_CASE(6) VS_CASE(7)
#undef VS_CASE
    default: e = sweep<K_PAIRS, CUT, DIEL>(a, L, R, ox, oy, oz, tile, full, relcnt, src, len, nt, nwarps); break;
  }

  // pairs evaluated: real ligand atoms of each lane's group x receptor atoms streamed; poses counted once
  // (by the CTA holding their group-0 item)
  unsigned npair = active ? (unsigned)__ldg(a.group_natoms + group) : 0u;
  npair = __reduce_add_sync(0xffffffffu, npair);
  const unsigned n0 = __popc(__ballot_sync(0xffffffffu, active && group == 0 && blockIdx.z == 0));
  if (lane == 0 && a.counters) {
    if (npair) atomicAdd(a.counters + 0, (unsigned long long)npair * (unsigned long long)len);
    if (n0) atomicAdd(a.counters + 1, (unsigned long long)n0);
  }
  red[warp][lane] = e;
  __syncthreads();
  if (warp == 0) {
    double sum = 0.0;
    for (int w = 0; w < nwarps; ++w) sum += red[w][lane];
    bool finish = active;
    if (active && a.n_chunks * a.nsplit > 1) {
      // the pose's energy is split over ligand groups (and list splits) held by several CTAs: write this
      // partial; the CTA that completes the pose adds all partials in a fixed order (deterministic) and
      // applies the epilogue (no separate finalize launch)
      const int np = a.n_chunks * a.nsplit;
      const int slot = (a.mixed ? group : chunk) * a.nsplit + blockIdx.z;
      a.partial[(size_t)item * np + slot] = sum;
      __threadfence();
      finish = atomicAdd(a.done + item, 1u) == (unsigned)(np - 1);
      if (finish) {
        __threadfence();
        sum = 0.0;
        for (int c = 0; c < np; ++c) sum += __ldcg(a.partial + (size_t)item * np + c);
        a.done[item] = 0u;  // ready for the next launch
      }
    }
    const float score = (float)sum;
    if (finish) {
      if (MODE == MODE_PLAIN) {
        const int pidx = a.uniform ? k * a.seg_stride + (a.perm ? __ldg(a.perm + k * a.seg_size + p) : p) : item;
        a.poses[pidx].t.w = score;
        if (a.orig) a.score_out[__ldg(a.orig + pidx)] = score;
      } else if (a.K > 1) {
        a.pscore[item] = score;                                  // best of K chosen by lsk_accept_kernel
      } else if (score < old_score) {                            // strict improvement (R16)
        PoseRec rr;
        rr.q = q;
        rr.t = make_float4(t.x, t.y, t.z, score);
        a.poses[jx] = rr;
      }
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
  const int warps = a.mixed ? 1 : (a.n_chunks > 1 ? GROUPS_PER_CTA : a.n_groups);
  dim3 grid(n_blocks, a.mixed ? 1 : a.n_chunks, a.nsplit), block(warps * 32);
  if (mode == MODE_PLAIN)
    return cutoff ? launch_diel<MODE_PLAIN, true>(a, dielectric, grid, block, st)
                  : launch_diel<MODE_PLAIN, false>(a, dielectric, grid, block, st);
  return cutoff ? launch_diel<MODE_LS, true>(a, dielectric, grid, block, st)
                : launch_diel<MODE_LS, false>(a, dielectric, grid, block, st);
}


}  // namespace vsk

namespace vsk {

// Parallel-neighbourhood Improve (N4): element j of segment k takes the best of its K proposals
// (strict <, lowest k on ties) if that is strictly better than itself.
__global__ void lsk_accept_kernel(const ScoreArgs a) {
  const int idx = blockIdx.x * blockDim.x + threadIdx.x;
  if (idx >= a.nseg * a.m) return;
  const int k = idx / a.m, jj = idx - k * a.m;
  const float* ps = a.pscore + ((size_t)k * a.m + jj) * a.K;
  int best = 0;
  for (int kk = 1; kk < a.K; ++kk)
    if (ps[kk] < ps[best]) best = kk;
  const int j = __ldg(a.J + k * a.m + jj);
  const int jx = k * a.P + j;
  PoseRec r = a.poses[jx];
  if (ps[best] < r.t.w) {
    float4 q = r.q, t = r.t;
    perturb(q, t, a.ls_trans, a.ls_rot, a.T, *a.seedp, (uint32_t)j, (uint32_t)__ldg(a.seg_spot + k), (uint32_t)a.g,
            TAG_LS, 2u * (uint32_t)(a.l * a.K + best));
    r.q = q;
    r.t = make_float4(t.x, t.y, t.z, ps[best]);
    a.poses[jx] = r;
  }
}

cudaError_t launch_lsk_accept(const ScoreArgs& a, cudaStream_t st) {
  const int n = a.nseg * a.m;
  lsk_accept_kernel<<<(n + 127) / 128, 128, 0, st>>>(a);
  return cudaGetLastError();
}

// Lanes = poses (warp-uniform ligand group, H-bond-specialised loop) unless the segment is short
// enough that (pose, group) items fill clearly more lanes (e.g. Improve's m = 51 or 13 poses).
int plan_uniform(ScoreArgs& a, int seg_size, long target_warps) {  // target: warps per spot
  a.seg_size = seg_size;
  a.fbps = (seg_size + POSES_PER_CTA - 1) / POSES_PER_CTA;
  const long lanes_pose = (long)a.fbps * POSES_PER_CTA * a.n_groups;
  const long items = (long)seg_size * a.n_groups;
  const long lanes_mixed = (items + POSES_PER_CTA - 1) / POSES_PER_CTA * POSES_PER_CTA;
  a.mixed = (GROUPS_PER_CTA == 1 && a.n_groups > 1 && lanes_mixed * 100 < lanes_pose * 95) ? 1 : 0;
  a.bps = a.mixed ? (int)(lanes_mixed / POSES_PER_CTA) : a.fbps;
  // split each spot's receptor list over up to 8 CTAs when a spot has few warps of work (Improve's m poses,
  // small populations).  The rule depends only on per-spot quantities, never on how many spots a launch
  // holds, so results are bitwise independent of the spot chunking and of the number of GPUs.
  const long warps_per_spot = (long)a.bps * (a.mixed ? 1 : a.n_chunks * GROUPS_PER_CTA);
  a.nsplit = 1;
  while (a.nsplit < 8 && warps_per_spot * a.nsplit < target_warps) a.nsplit *= 2;
  return a.bps;
}

}  // namespace vsk
