// vs_kernels.cuh -- launch-side declarations shared by vs_cells.cu, vs_pop.cu, vs_api.cu.
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

#include "vs_device.cuh"

namespace vsk {

// ---------------------------------------------------------------- programmatic dependent launch (PDL)
// The kernels of a run's per-stream chain (init / combine / popsort / best and the three scoring kernels) are
// launched with programmatic stream serialization, so a kernel may be scheduled while its predecessor drains; its
// first statement (griddepcontrol.wait) blocks until the predecessor grid has completed and its memory is
// visible, so only launch latency is overlapped (small config 25.8 -> 24.9 ms / step).  With VS_PDL_TRIGGER the
// chain kernels also signal launch_dependents at entry; measured on B200 that lets waiting dependents hold SM
// slots the other spot-group streams need (medium 602 -> 785 ms / step), so it is off.
#ifndef VS_PDL
#define VS_PDL 1
#endif
#ifndef VS_PDL_TRIGGER
#define VS_PDL_TRIGGER 0
#endif

// trig (runtime, per launch): also signal launch_dependents at entry, so the next kernel of the chain is scheduled
// while this one runs and starts the instant it completes.  Used for latency-bound runs (few spots: the GPU has
// idle slots for the waiting CTAs); for full runs the waiting CTAs would hold SM slots the other streams need.
__device__ __forceinline__ void pdl_enter(int trig = 0) {
#if VS_PDL
  asm volatile("griddepcontrol.wait;\n" ::: "memory");
#if VS_PDL_TRIGGER
  trig = 1;
#endif
  if (trig) asm volatile("griddepcontrol.launch_dependents;\n" ::: "memory");
#endif
}

template <typename... KP, typename... AP>
cudaError_t launch_chain(void (*k)(KP...), dim3 grid, dim3 block, size_t smem, cudaStream_t st, AP... args) {
#if VS_PDL
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  at[0].val.programmaticStreamSerializationAllowed = 1;
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = grid;
  cfg.blockDim = block;
  cfg.dynamicSmemBytes = smem;
  cfg.stream = st;
  cfg.attrs = at;
  cfg.numAttrs = 1;
  return cudaLaunchKernelEx(&cfg, k, args...);
#else
  k<<<grid, block, smem, st>>>(args...);
  return cudaGetLastError();
#endif
}

enum ScoreMode : int { MODE_PLAIN = 0, MODE_LS = 1 };

// ---------------------------------------------------------------- scoring (vs_cells.cu)
// Work unit = chunk of up to CH_ITEMS transformed ligand atoms ("items": one ligand atom of one pose),
// spatially sorted per spot; the chunk streams only the cell rows of the spot's cell-sorted list
// within rc of its bounding box.
#ifndef VS_CELL_MERGE
#define VS_CELL_MERGE 0  // 1: every ligand atom in class 1 (one item order, all slot pairs H-bond pairs)
#endif
#ifndef VS_CELL_G
#define VS_CELL_G 0  // 0: cells per axis chosen per context from its list splits (vs_api.cu cell_grid); > 0 forces it
#endif
#ifndef VS_CELL_EXACTX
#define VS_CELL_EXACTX 0  // exact-x trim of row runs: redundant with the per-pair atom test (VS_CELL_PPCULL), measured 1.4 % slower
#endif
constexpr int CELL_GMAX = 24;                      // largest list grid per spot: G^3 cells over [-R, R]^3, G <= 24
constexpr int CELL_SORT_MAX = 16384;               // longest list cell-sorted in shared memory (128 KB keys)
constexpr int CELL_KP = 2;                         // packed float2 item pairs per lane of the default pair kernel
constexpr int CH_ITEMS = 2 * CELL_KP * 32;         // items per chunk (one warp) of the default pair kernel
constexpr int CELL_NSPLIT = 4;                     // most canonical receptor-list splits (item energy (e0+e1)+(e2+e3))
#ifndef VS_CELL_BATCH
#define VS_CELL_BATCH 64
#endif
constexpr int CELL_BATCH = VS_CELL_BATCH;          // receptor atoms per staging buffer (2 per lane per 64)
constexpr int CELL_MAXRUN = CELL_GMAX * CELL_GMAX; // one run per cell row at most
constexpr int MORTON_BITS = 4;                     // item sort grid: 16^3 cells over the spot region
constexpr int MORTON_BINS = 1 << (3 * MORTON_BITS);

struct CellArgs {
  // receptor lists (per spot) and the cell start table [n_spots][cg^3 + 1] (uint16 list positions; a
  // cell-sorted list has <= CELL_SORT_MAX < 2^16 atoms; cells[s][0] == 0xFFFF: not cell-sorted -> streamed whole)
  const RecAtom* lists;
  const int* list_off;
  const int* list_len;
  const uint16_t* cells;
  float cR, ch, cinv_h;      // grid half-width (A), cell edge, 1 / edge
  int cg;                    // cells per axis of the list grid (a context property; S divides it)
  // ligand (input order)
  const float4* ligx;        // local x, y, z (centred), w = class (0: class 0; 1: class 1, donor / acceptor; 2: class 1, no role)
  const float4* ligp;        // es_i, c12_i, c6_i, donor_i
  const int* lig_rank;       // rank of the atom within its class
  int n_lig, nn, nh;         // atoms; in class 0 / class 1 (H-bond role) for this launch (merged: 0 / n_lig)
  int merged;                // every atom in class 1, rank = atom index (a KP = 1 launch of a ligand with roles)
  // launch shape (speed only, never results): kp packed item pairs per lane (1 or 2), H of them H-bond pairs (the
  // first kp - H pairs hold class 0 only), chunk capacities cn = 64 kp items, chb = 64 H class-1 items (w: 1)
  int kp, H, cn, chb, w;
  int nsplit;                // canonical list splits S (1, 2, 4) of the context, one warp each: the split tree
                             // (e0 + e1) + (e2 + e3) of an item's split energies defines the result
  const float4* shift;       // added to t + R l (all-pairs: 0 -- lists are spot-relative)
  float W, inv_hm;           // item sort grid: [-W, W]^3, 16 cells per axis
  int cut;                   // cutoff mode (cell culling, spatial item sort)
  // segments (one spot each)
  int nseg;
  const int* seg_spot;
  int uniform, seg_size;     // uniform: every segment has seg_size poses
  const int* pose_prefix;    // non-uniform: [nseg + 1]
  const int* chunk_prefix;   // non-uniform: [nseg + 1]
  int nch_u;                 // uniform: chunks per segment
  // poses
  int mode;                  // MODE_PLAIN / MODE_LS
  PoseRec* poses;            // PLAIN: segment k pose p at k * seg_stride + p (uniform) or pose_prefix[k] + p;
                             // LS: the population X (k * P + j)
  int seg_stride;
  const int* orig;           // PLAIN non-uniform: original index of each pose -> score_out
  float* score_out;
  const int* J;
  int m, P, K;
  const uint64_t* seedp;
  int g, l;
  float ls_trans, ls_rot, T;
  // launch scratch
  PoseRec* pbuf;             // [launch poses] the pose scored (LS: the proposal, t.w = score of X[j])
  float4* items;             // [launch items] per segment: class-0 items then class-1 items, each spatially sorted
  double* E;                 // [nsplit][launch items] per-item energies of each split
  long long E_stride;
  float r2min, rc, rc2, inv_rc2;
  float hbC, hbD;
  unsigned long long* counters;  // [0] pairs evaluated, [1] poses, [2] workload pairs, [3] pairs within rc (census)
  int census;                // count the pairs within rc (a separate pair-kernel instantiation; same results)
  // instrumentation: pair-kernel launch intervals (globaltimer) in slot kt_slot of the run's region at *kt_base
  unsigned long long* kt;
  const unsigned long long* kt_base;
  int kt_slot, kt_cap;
  int trig;                  // PDL early trigger (latency-bound runs, pdl_enter)
};
constexpr int KT_WORDS = 3;  // per launch slot: ~start, end, sum of warp durations (ns)

// Chunks of a segment of seg_n poses: class-1 items (H-bond role) fill at most cap1 = 64 H slots (the last H
// slot pairs of each lane), class-0 items the other slots and any H-bond slot left over; a chunk takes the
// same spatial quantile of both classes, so it must hold ceil(Nn / c) + ceil(Nh / c) <= cap items.
__host__ __device__ inline int cell_chunks(int seg_n, int nn, int nh, int cap, int cap1) {
  if (seg_n <= 0) return 0;
  const long long Nn = (long long)seg_n * nn, Nh = (long long)seg_n * nh;
  long long c = (Nn + Nh + cap - 1) / cap;
  if (Nh > 0) c = c > (Nh + cap1 - 1) / cap1 ? c : (Nh + cap1 - 1) / cap1;
  while ((Nn + c - 1) / c + (Nh + c - 1) / c > cap || (Nh + c - 1) / c > cap1) ++c;
  return (int)c;
}

cudaError_t launch_cell_sort(const RecAtom* lists, RecAtom* out, const int* off, const int* len, int n_spots, uint16_t* cells,
                             int G, float R, float inv_h, cudaStream_t st);
// K1 + K2 + K3 of one scoring call; n_blocks2 = pair-kernel grid (upper bound when non-uniform)
cudaError_t launch_cell_score(const CellArgs& a, int dielectric, long long n_poses, int n_blocks2, cudaStream_t st);
cudaError_t launch_kt_advance(unsigned long long* kt_base, int slots, cudaStream_t st);
cudaError_t launch_cell_scan(const int* counts, int n, int nn, int nh, int cn, int chb, int* pose_prefix,
                             int* chunk_prefix, int* cursor, cudaStream_t st);

// launchers (return cudaError_t of the launch)
cudaError_t launch_init(PoseRec* S, int n_sel, int P, const int* seg_spot, const uint64_t* seedp, float T, int trig,
                        cudaStream_t st);
cudaError_t launch_combine(const PoseRec* S, PoseRec* C, int n_sel, int P, const int* seg_spot, const uint64_t* seedp, int g,
                           float p_mut, float mut_trans, float mut_rot, float T, int trig, cudaStream_t st);
// sort (score, index) per segment: mode 0: select best m indices -> J;
// mode 1: sort S -> S_out; mode 2: include: best P of S ++ C -> S_out
cudaError_t launch_popsort(int mode, const PoseRec* S, const PoseRec* C, PoseRec* S_out, int* J, int n_sel, int P,
                           int m, int trig, cudaStream_t st);
cudaError_t launch_best(const PoseRec* S, int n_sel, int P, float* best_pose, float* best_score, cudaStream_t st);
cudaError_t launch_build_lists(const float4* rec, const float4* rprm, int n_rec, const float4* spot_c, int n_spots,
                               float reach2, const int* off, int* len, RecAtom* lists, int count_only,
                               cudaStream_t st);
cudaError_t launch_philox(int64_t n, const uint4* ctr, uint2 key, uint4* out, cudaStream_t st);
// vs_score_poses helpers
cudaError_t launch_validate(int64_t n, const int32_t* spot, const float* q, const float* t, int n_spots, float T,
                            int cutoff, int* valid, int* counts, float* score_out, cudaStream_t st);
cudaError_t launch_scatter(int64_t n, const int32_t* spot, const float* q, const float* t, const int* valid,
                           int* cursor, PoseRec* sorted, int* orig, cudaStream_t st);

}  // namespace vsk
