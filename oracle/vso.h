/* oracle/vso.h -- fp64 CPU ORACLE of the metaheuristic virtual-screening hot path.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and the
 * cpu_baseline / --impl reference legs of bench.py may load this library.
 * The product path (paper_conf_ppopp_imbernoncg16_b200) never calls it.
 * It shares no source, header, table or constant generator with the CUDA
 * path (include/vs.h, paper_conf_ppopp_imbernoncg16_b200/csrc/).
 *
 * It is the plain definition written out:
 *   - scoring: brute force over ALL ligand x receptor atom pairs in fp64
 *     (§2.1 P:55 "Coulomb ... and the Lennard-Jones potentials",
 *     §1 P:23 "computations between pairs of atoms in the protein and the
 *     ligand"; pair terms per DESIGN.md readings R1-R8);
 *   - metaheuristic: Algorithm 1 (§3.1) step by step --
 *     Initialize, End, Select, Combine, Improve, Include -- with the T4
 *     parameters and the Philox streams of DESIGN.md R23.
 * Pose generation uses IEEE fp32 single operations in the written order
 * (reading R24) so that its bytes can be compared with the GPU's; decisions
 * taken on scores (accept, sorts) compare the fp64 scores rounded to fp32,
 * the kernel's precision (R26).
 *
 * ABI mirrors include/vs.h with the prefix vso_ (host only).
 */
#ifndef VSO_H
#define VSO_H
#include <stdint.h>
#ifdef __cplusplus
extern "C" {
#endif

typedef struct vso_ctx vso_ctx;
typedef enum { VSO_OK = 0, VSO_ERR_INVALID_ARGUMENT = 1, VSO_ERR_POSE_OUT_OF_REGION = 2,
               VSO_ERR_ZERO_QUATERNION = 3, VSO_ERR_CUDA = 4, VSO_ERR_OUT_OF_MEMORY = 5,
               VSO_ERR_UNSUPPORTED = 6 } vso_status;

typedef struct {
  float coulomb_k; int dielectric; float eps_r; float cutoff; float region_half_width;
  float hb_eps, hb_r0; float r2_min;
  int n_types; const float* type_sigma; const float* type_eps; const int* type_hb_role;
} vso_score_params;

typedef struct {
  int population, generations, ls_steps;
  float improve_frac, p_mut, mut_trans, mut_rot, ls_trans, ls_rot;
  int ls_neighbours;   /* K proposals per Improve step, best-of-K accepted; 1 = hill climbing */
} vso_mh_params;

void        vso_score_params_default(vso_score_params* out);
vso_status  vso_mh_preset(int m, vso_mh_params* out);
vso_status  vso_create(const float* rec_xyz, const float* rec_q, const int32_t* rec_type, int32_t n_rec,
                       const float* lig_xyz, const float* lig_q, const int32_t* lig_type, int32_t n_lig,
                       const float* spot_xyz, int32_t n_spots, const vso_score_params* sp,
                       int32_t cuda_device, vso_ctx** out);
vso_status  vso_score_poses(vso_ctx* c, int64_t n, const int32_t* spot, const float* quat_wxyz,
                            const float* trans, float* score_out);
vso_status  vso_score_poses_d(vso_ctx* c, int64_t n, const int32_t* spot, const float* quat_wxyz,
                              const float* trans, double* score_out);
vso_status  vso_run(vso_ctx* c, const vso_mh_params* mp, uint64_t seed, int32_t n_sel,
                    const int32_t* spot_ids, float* best_pose_out, float* best_score_out);
vso_status  vso_run_d(vso_ctx* c, const vso_mh_params* mp, uint64_t seed, int32_t n_sel,
                      const int32_t* spot_ids, float* best_pose_out, double* best_score_out);
void        vso_destroy(vso_ctx* c);
const char* vso_last_error(void);
int         vso_abi_version(void);

/* ---- building blocks exposed for pins and lockstep tests --------------- */
void     vso_set_threads(int n);          /* OpenMP threads; <= 0 -> runtime default */
int      vso_get_threads(void);
void     vso_philox4x32_10(const uint32_t ctr[4], const uint32_t key[2], uint32_t out[4]);
float    vso_u01(uint32_t w);
float    vso_v11(uint32_t w);
/* score of one pose without the ABI region check (fp64) */
double   vso_score_one(const vso_ctx* c, int32_t spot, const float q[4], const float t[3]);
/* ligand coordinates relative to the fp32 centroid, as used by the pose transform */
void     vso_ligand_local(const vso_ctx* c, float* out_xyz /*[n_lig][3]*/);
uint64_t vso_pairs_evaluated(const vso_ctx* c);   /* running count of (i,j) pairs visited */
uint64_t vso_pairs_within(const vso_ctx* c);      /* running count of visited pairs with r^2 < rc^2 (all in all-pairs mode) */
/* pose = float[7] = (w,x,y,z,tx,ty,tz) */
void vso_init_pose(const vso_ctx* c, uint64_t seed, int32_t spot, int32_t i, float pose_out[7]);
void vso_combine_child(const vso_ctx* c, const vso_mh_params* mp, uint64_t seed, int32_t spot,
                       int32_t g, int32_t j, const float* S_sorted /*[P][7]*/, float pose_out[7]);
/* Select (R13): the parents (sorted-population ranks) of child j of generation g at `spot` */
void vso_select_parents(const vso_mh_params* mp, uint64_t seed, int32_t spot, int32_t g, int32_t j,
                        int32_t* p1_out, int32_t* p2_out);
void vso_ls_proposal(const vso_ctx* c, const vso_mh_params* mp, uint64_t seed, int32_t spot,
                     int32_t g, int32_t l, int32_t j, const float pose_in[7], float pose_out[7]);
/* proposal k (0 <= k < ls_neighbours) of Improve step l for individual j */
void vso_ls_proposal_k(const vso_ctx* c, const vso_mh_params* mp, uint64_t seed, int32_t spot,
                       int32_t g, int32_t l, int32_t k, int32_t j, const float pose_in[7], float pose_out[7]);
int32_t vso_improve_count(const vso_mh_params* mp);          /* m of Improve */
/* J = indices of the best m of scores[P] by (score, index) */
void vso_select_improve(const double* scores, int32_t P, int32_t m, int32_t* J_out);
/* stable (mu+lambda): first P of sort(S ++ C) by score; out_origin[k] = index into S++C */
void vso_include(const double* sS, const double* sC, int32_t P, int32_t* out_origin);

#ifdef __cplusplus
}
#endif
#endif
