// vs_kernels.cuh -- launch-side declarations shared by vs_score.cu, vs_pop.cu, vs_api.cu.
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

#include "vs_device.cuh"

namespace vsk {

#ifndef VS_KPAIRS
#define VS_KPAIRS 3
#endif
constexpr int K_PAIRS = VS_KPAIRS;   // slot pairs per thread: one float2 lane-pair per FFMA2
constexpr int K_SLOTS = 2 * K_PAIRS; // ligand atoms per thread (register blocking)
#ifndef VS_GPC
#define VS_GPC 1
#endif
constexpr int GROUPS_PER_CTA = VS_GPC;  // warps (ligand-atom groups) per CTA at most
constexpr int POSES_PER_CTA = 32;   // one pose per lane
#ifndef VS_TILE
#define VS_TILE 128
#endif
#ifndef VS_NSTAGE
#define VS_NSTAGE 4
#endif
constexpr int TILE = VS_TILE;       // receptor atoms per shared-memory stage (32 B each)
constexpr int NSTAGE = VS_NSTAGE;   // bulk-copy ring depth

enum ScoreMode : int { MODE_PLAIN = 0, MODE_LS = 1 };

// Per-spot lists are sorted by distance from the spot centre; shell[s][b] = number of list atoms with
// |r| < (b + 1) * SHELL_DR.  A warp whose ligand atoms all lie within R_w of the spot centre streams only
// the atoms with |r| < R_w + rc (the others are provably beyond the cutoff of every pair).
constexpr int NSHELL = 256;
constexpr float SHELL_DR = 0.125f;   // A: table covers 32 A
constexpr int SORT_MAX = 4096;       // longest list sorted in shared memory (32 KB of keys)

// Work decomposition of one scoring launch: segments (one spot each) of poses,
// split into 32-pose blocks; blockIdx.y = ligand group chunk.
struct ScoreArgs {
  // receptor lists (per spot) and ligand slots
  const RecAtom* lists;
  const int* list_off;
  const int* list_len;
  const float4* shift;       // added to t + R l (all-pairs: c_s - c0; cutoff: 0)
  const int* shell;          // cutoff mode: [n_spots][NSHELL] prefix counts of the distance-sorted lists
  const int* group_natoms;   // real (non-padding) ligand atoms per group, for pair accounting
  const LigSlot* lig;
  int n_groups;              // ligand groups of K_SLOTS slots
  int hb_base, hb_extra;     // group g holds hb_base + (g < hb_extra) H-bond slot pairs, at its end
  int hb_max;                // max over groups
  int mixed;                 // 1: lanes map to (pose, group) items of a segment (1-warp CTAs, grid.y = 1)
  int n_chunks;              // ceil(n_groups / GROUPS_PER_CTA)
  int nsplit;                // receptor-list splits per (pose block, group) (grid.z); partial sums when > 1
  int n_lig;                 // real ligand atoms (pair accounting)
  float r2min, rc, rc2, inv_rc2; // rc, rc2 = +inf in all-pairs mode
  float hbC, hbD;
  // segments
  int nseg;
  const int* seg_spot;       // [nseg] global spot id
  int uniform;               // 1: every segment has seg_size poses
  int seg_size, bps;         // uniform: poses per segment, scoring blocks per segment
  int fbps;                  // uniform: 32-pose blocks per segment
  const int* blk_prefix;     // non-uniform: [nseg+1]
  const int* pose_prefix;    // non-uniform: [nseg+1]
  // PLAIN
  PoseRec* poses;            // segment k pose p at k*seg_stride + p (uniform) or pose_prefix[k] + p
  int seg_stride;
  const int* orig;           // optional: original index of each pose -> score_out
  const int* perm;           // optional (uniform PLAIN): scoring order of segment k, [nseg][seg_size]
  float* score_out;
  double* partial;           // n_chunks * nsplit > 1: [items][n_chunks * nsplit] partial energies
  unsigned* done;            // [items] contributions received (reset to 0 by the completing CTA)
  // LS (Improve step): X[k*P + J[k*m + jj]] perturbed, scored, accepted if better
  const int* J;
  int m, P;
  int K;                     // proposals per Improve step (segment item p: element p / K, proposal p % K)
  float* pscore;             // K > 1: proposal scores [nseg][m][K], accepted by lsk_accept_kernel
  const uint64_t* seedp;      // run seed in device memory (graph replays need no new parameters)
  int g, l;
  float ls_trans, ls_rot, T;
  unsigned long long* counters;  // [0] pairs, [1] poses
};

// launchers (return cudaError_t of the launch)
cudaError_t launch_score(const ScoreArgs& a, int mode, bool cutoff, int dielectric, int n_blocks, cudaStream_t st);
cudaError_t launch_lsk_accept(const ScoreArgs& a, cudaStream_t st);
// lane mapping for a uniform launch of nseg segments of seg_size poses: sets mixed / bps / fbps;
// returns the number of scoring blocks
int plan_uniform(ScoreArgs& a, int seg_size, long target_warps);
cudaError_t launch_init(PoseRec* S, int n_sel, int P, const int* seg_spot, const uint64_t* seedp, float T, cudaStream_t st);
cudaError_t launch_combine(const PoseRec* S, PoseRec* C, int n_sel, int P, const int* seg_spot, const uint64_t* seedp, int g,
                           float p_mut, float mut_trans, float mut_rot, float T, cudaStream_t st);
// sort (score, index) per segment: mode 0: select best m indices -> J;
// mode 1: sort S -> S_out; mode 2: include: best P of S ++ C -> S_out
cudaError_t launch_popsort(int mode, const PoseRec* S, const PoseRec* C, PoseRec* S_out, int* J, int n_sel, int P,
                           int m, cudaStream_t st);
cudaError_t launch_best(const PoseRec* S, int n_sel, int P, float* best_pose, float* best_score, cudaStream_t st);
cudaError_t launch_build_lists(const float4* rec, const float4* rprm, int n_rec, const float4* spot_c, int n_spots,
                               float reach2, const int* off, int* len, RecAtom* lists, int count_only,
                               cudaStream_t st);
// sort every cutoff list by distance from its spot centre (stable) and fill the shell table
cudaError_t launch_sort_lists(RecAtom* lists, RecAtom* tmp, const int* off, const int* len, int n_spots, int* shell,
                              cudaStream_t st);
cudaError_t launch_philox(int64_t n, const uint4* ctr, uint2 key, uint4* out, cudaStream_t st);
// vs_score_poses helpers
cudaError_t launch_validate(int64_t n, const int32_t* spot, const float* q, const float* t, int n_spots, float T,
                            int cutoff, int* valid, int* counts, float* score_out, cudaStream_t st);
cudaError_t launch_scan(const int* counts, int n, int* pose_prefix, int* blk_prefix, int* cursor, cudaStream_t st);
cudaError_t launch_scatter(int64_t n, const int32_t* spot, const float* q, const float* t, const int* valid,
                           int* cursor, PoseRec* sorted, int* orig, cudaStream_t st);

}  // namespace vsk
