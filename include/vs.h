/* include/vs.h -- C ABI of the B200-native virtual-screening hot path.
 *
 * What it computes (PAPER.md = Imbernon, Cecilia, Gimenez, PMAM'16;
 * "P:N" = line N of PAPER.md; "Rn" = reading n in DESIGN.md §3):
 *   - the scoring function of a rigid ligand pose placed near a receptor
 *     spot: a sum over all ligand-atom x receptor-atom pairs of
 *     electrostatic, Lennard-Jones and hydrogen-bond terms
 *     ("computations between pairs of atoms in the protein and the
 *     ligand"; P:55 Coulomb + Lennard-Jones; P:84 spots, conformations;
 *     pair terms R1-R8);
 *   - the metaheuristic of Algorithm 1 (Initialize, End, Select,
 *     Combine, Improve, Include) run independently at every spot (P:84,
 *     P:140), with the Table 4 parameters as presets.
 *
 * Conventions (all functions):
 *   - extern "C", never throw, never abort; a non-OK status leaves a
 *     thread-local message readable with vs_last_error().
 *   - The caller owns every buffer it passes.  vs_create deep-copies its
 *     inputs; outputs go to caller-sized buffers; on error the output
 *     buffers are unspecified and vs_create returns *out = NULL.
 *   - A ctx is bound to one CUDA device and used by one host thread at a
 *     time; several ctx may share a device.
 *   - After VS_ERR_CUDA a ctx is poisoned: every later call except
 *     vs_destroy returns VS_ERR_CUDA.
 *   - Units: Angstrom, elementary charge, kcal/mol.  Arrays are row-major
 *     fp32 / int32 host arrays unless a name starts with d_ (device memory
 *     of the ctx's device).
 */
#ifndef VS_H
#define VS_H
#include <stdint.h>
#ifdef __cplusplus
extern "C" {
#endif

#define VS_ABI_VERSION 4

#if defined(__GNUC__)
#define VS_API __attribute__((visibility("default")))
#else
#define VS_API
#endif

typedef struct vs_ctx vs_ctx; /* opaque; owned by the library */

typedef enum {
  VS_OK = 0,
  VS_ERR_INVALID_ARGUMENT = 1,   /* NULL pointer, bad count, bad type id, non-finite input */
  VS_ERR_POSE_OUT_OF_REGION = 2, /* cutoff mode: |t_k| > region_half_width (R10) */
  VS_ERR_ZERO_QUATERNION = 3,    /* quaternion with zero norm */
  VS_ERR_CUDA = 4,               /* CUDA runtime failure (ctx poisoned) */
  VS_ERR_OUT_OF_MEMORY = 5,      /* host or device allocation failed */
  VS_ERR_UNSUPPORTED = 6         /* valid request this build does not implement */
} vs_status;

/* Scoring-function parameters.  vs_score_params_default() fills:
 *   coulomb_k 332.0636 (R2), dielectric 0 = eps(r) = 4r (R3), eps_r 1,
 *   cutoff 12 A with electrostatic shift (1 - r^2/rc^2)^2 (R6),
 *   region_half_width 3 A (R10), hb_eps 5 kcal/mol, hb_r0 1.9 A (R5),
 *   r2_min 0.01 A^2 (R7), n_types 0 = built-in 7-type table:
 *     id: 0 C, 1 N, 2 O, 3 S, 4 H, 5 HD (polar H), 6 X (dummy)
 *     sigma 3.400 3.250 2.960 3.564 2.650 1.069 0
 *     eps   0.1094 0.170 0.210 0.250 0.0157 0.0157 0
 *     role  -  acc  acc  -  -  donor  -       (1 donor, 2 acceptor)
 * cutoff <= 0 or +inf selects all-pairs mode (the paper's brute-force
 * reading); a finite cutoff selects per-spot binned lists, exact for
 * every pose inside the region (R10).  dielectric 1 (constant eps_r,
 * E = k qi qj / (eps_r r)) is accepted. */
typedef struct {
  float coulomb_k;
  int dielectric;
  float eps_r;
  float cutoff;
  float region_half_width;
  float hb_eps, hb_r0;
  float r2_min;
  int n_types;                /* 0 -> built-in table; else 1..64 entries below */
  const float* type_sigma;    /* [n_types] A   (>= 0) */
  const float* type_eps;      /* [n_types] kcal/mol (>= 0) */
  const int* type_hb_role;    /* [n_types] 0 none, 1 donor, 2 acceptor */
  int list_splits;            /* canonical receptor-list splits S: 1, 2 or 4; 0 (default) = by the spot count
                                 (<= 96 spots: 4, <= 200: 2, else 1).  The GPU sums each
                                 split's pairs in fp32 and combines the split energies of an atom by the fixed fp64
                                 tree (e0 + e1) + (e2 + e3): a summation order, so scores differ from S = 1 at fp32
                                 rounding (all within the tolerance).  For a given S a pose's score is the same from
                                 every entry point and launch, whatever the spot count or GPU count of the run; S > 1
                                 gives latency-bound runs (few spots per GPU) up to S x more parallel work.  Not
                                 part of the method: the oracle ignores it. */
} vs_score_params;

/* Metaheuristic parameters (Algorithm 1; Table 4).
 * population P (1..2048; >= 2 when generations > 0), generations G >= 0
 * (End condition, R20), ls_steps L >= 0 with L x ls_neighbours <= 2^23
 * (the LS Philox counter, R23) (Improve, R16), improve_frac f in
 * [0,1] (Table 4 "% of elements to be improved"; m = clamp(round(f*P),1,P)
 * elements, R17), p_mut in [0,1] (R15), step sizes >= 0 (A, radians-ish
 * quaternion increments). */
typedef struct {
  int population, generations, ls_steps;
  float improve_frac, p_mut, mut_trans, mut_rot, ls_trans, ls_rot;
  int ls_neighbours;  /* K in [1, 64] proposals per Improve step scored together, the best replaces the
                         element if strictly better; 1 = first-improvement hill climbing */
} vs_mh_params;

VS_API void vs_score_params_default(vs_score_params* out);

/* m = 1..4 -> M1..M4 of Table 4:
 *   M1 GA: P 64, f 0;  M2: P 64, f 1, L 8;  M3: P 64, f 0.2, L 8;
 *   M4: P 1024, G 0, f 1, L 8 ("only one step").
 *   G = 50 for M1-M3 (the paper does not report it, R22); p_mut 0.1,
 *   mut 1.0 A / 0.25, ls 0.5 A / 0.10, ls_neighbours 1.
 * Returns VS_ERR_INVALID_ARGUMENT for another m or out == NULL. */
VS_API vs_status vs_mh_preset(int m, vs_mh_params* out);

/* Builds a scoring context on CUDA device `cuda_device`.
 *   rec_xyz [n_rec][3], rec_q [n_rec], rec_type [n_rec]  receptor atoms
 *   lig_xyz [n_lig][3], lig_q [n_lig], lig_type [n_lig]  ligand atoms, 1 <= n_lig <= 256
 *   spot_xyz [n_spots][3]                                spot centres (R9)
 *   sp: NULL -> defaults.
 * The ligand is centred on its centroid (fp64 sum, rounded to fp32 once;
 * l_i = lig_xyz_i - centroid in fp32, R11).  In cutoff mode the per-spot
 * receptor lists (atoms within T*sqrt(3) + max|l_i| + rc + 0.01 A of the
 * spot centre, R10) are built on the device here.
 * Errors: VS_ERR_INVALID_ARGUMENT (NULL / counts / type ids / non-finite /
 * bad params), VS_ERR_CUDA, VS_ERR_OUT_OF_MEMORY.  *out = NULL on error. */
VS_API vs_status vs_create(const float* rec_xyz, const float* rec_q, const int32_t* rec_type, int32_t n_rec,
                    const float* lig_xyz, const float* lig_q, const int32_t* lig_type, int32_t n_lig,
                    const float* spot_xyz, int32_t n_spots, const vs_score_params* sp, int32_t cuda_device,
                    vs_ctx** out);

/* Scores n poses (host buffers; synchronous).
 *   spot [n]         spot id of each pose (0 <= id < n_spots)
 *   quat_wxyz [n][4] rotation quaternion (w,x,y,z); need not be unit (R11), must be non-zero
 *   trans [n][3]     translation of the ligand centroid relative to the spot centre
 *   score_out [n]    score in kcal/mol (fp32)
 * x_i = c_spot + t + R(q) l_i;  score = sum_i sum_j e(i, j).
 * n == 0 is a no-op.  Errors: VS_ERR_INVALID_ARGUMENT (NULL, n < 0, bad
 * spot id, non-finite), VS_ERR_ZERO_QUATERNION, VS_ERR_POSE_OUT_OF_REGION
 * (cutoff mode only), VS_ERR_CUDA. */
VS_API vs_status vs_score_poses(vs_ctx* c, int64_t n, const int32_t* spot, const float* quat_wxyz, const float* trans,
                         float* score_out);

/* Same on device buffers, asynchronous with respect to `cuda_stream` (a
 * cudaStream_t; NULL = legacy default stream): the work is ordered after
 * everything enqueued on `cuda_stream` before the call, and later work on
 * `cuda_stream` is ordered after it (it runs on the ctx's own stream, joined
 * by events, so calls of one ctx never overlap each other, whatever streams
 * the caller uses).  Poses that fail validation get a NaN score instead of
 * an error status (no host round trip). */
VS_API vs_status vs_score_poses_device(vs_ctx* c, int64_t n, const int32_t* d_spot, const float* d_quat,
                                const float* d_trans, float* d_score, void* cuda_stream);

/* Runs the metaheuristic independently at n_sel spots (synchronous).
 *   spot_ids [n_sel] global spot ids (NULL -> all spots, n_sel must be 0 or
 *            n_spots); the id keys the Philox streams (R23), so a spot's
 *            result does not depend on which call / GPU / chunk ran it.
 *   best_pose_out [n_sel][7] = (w,x,y,z,tx,ty,tz) of the best individual
 *   best_score_out [n_sel]   its score (fp32, kcal/mol)
 * Errors: VS_ERR_INVALID_ARGUMENT (params, ids), VS_ERR_CUDA, VS_ERR_OUT_OF_MEMORY. */
VS_API vs_status vs_run(vs_ctx* c, const vs_mh_params* mp, uint64_t seed, int32_t n_sel, const int32_t* spot_ids,
                 float* best_pose_out, float* best_score_out);

/* Same, asynchronous with respect to `cuda_stream` (ordered after prior work
 * on it, later work on it ordered after the run; NULL = legacy default
 * stream); outputs in device memory.  spot_ids is a HOST array (validated
 * on the host, copied before the call returns).  The run itself executes on
 * the ctx's own streams (a CUDA graph from the second identical call on), so
 * calls of one ctx are serialised whatever streams the caller passes. */
VS_API vs_status vs_run_async(vs_ctx* c, const vs_mh_params* mp, uint64_t seed, int32_t n_sel, const int32_t* spot_ids,
                       float* d_best_pose, float* d_best_score, void* cuda_stream);

VS_API void vs_destroy(vs_ctx* c); /* NULL-safe; synchronises the ctx's device work */

/* Device memory of destroyed contexts is cached per device and handed to later contexts of the process (context
 * create / destroy then cost ~1 ms instead of tens of ms of cudaMalloc / cudaFree).  The cache holds at most
 * VS_POOL_CACHE_MB MiB per device (environment, read once; default 8192).  vs_release_cached_memory returns the
 * cached blocks of `cuda_device` (< 0: of every device) to the driver; live contexts keep theirs.  Thread-safe.
 * Errors: VS_ERR_INVALID_ARGUMENT (no such device). */
VS_API vs_status vs_release_cached_memory(int32_t cuda_device);

/* Environment variables read at vs_create (speed experiments only: no result depends on them beyond fp32 summation
 * order, and only VS_CELL_GRID changes that order):
 *   VS_GRAPHS=0             never capture CUDA graphs (plain launches, e.g. for profilers)
 *   VS_FILL_WARPS=n         scoring rounds with fewer pair-kernel warps than n use KP = 1 chunks (default 4096)
 *   VS_CELL_GRID=g          cells per axis of the per-spot list grid, 4..24, a multiple of list_splits (default 18
 *                           for 1-2 list splits, 20 for 4; changes the list order inside a cell row, hence rounding)
 *   VS_SHAPE=1|2            force the chunk shape KP
 *   VS_DIRECT_GROUP_SPOTS=n spots per stream group at least in un-graphed runs (default 16)
 *   VS_CELL_MERGE=0|1       one item class for every launch (default 0; KP = 1 launches merge anyway)
 *   VS_TRIGGER_SPOTS=n      runs of at most n spots use the PDL early trigger (default 0: off)
 *   VS_POOL_CACHE_MB=n      device memory cache cap (above) */
VS_API const char* vs_last_error(void);
VS_API int vs_abi_version(void);

/* ---- instrumentation ---------------------------------------------------- */
typedef struct {
  uint64_t kernel_launches;  /* all kernels this ctx launched */
  uint64_t score_launches;   /* scoring-kernel launches (plain + fused local search) */
  uint64_t poses_scored;     /* poses scored (incl. local-search proposals) */
  uint64_t pairs;            /* workload atom pairs: n_lig x list length (n_rec in all-pairs mode) per scored pose */
  double score_ms;           /* summed CUDA-event time of scoring launches (timing enabled) */
  uint64_t timed_launches;   /* launches covered by score_ms */
  uint64_t pairs_evaluated;  /* pairs the pair kernel evaluated: item slots x receptor atoms swept for them
                                (< pairs in cutoff mode: cell and slot-pair culling skip atoms beyond rc) */
  uint64_t pairs_within;     /* pairs within the cutoff, r^2 < rc^2 (census launches only, VS_TIMING_CENSUS):
                                the interactions that contribute to the scores; all-pairs mode: = pairs */
  double pair_busy_ms;       /* VS_TIMING_KERNEL: length of the union of the pair kernel's launch intervals */
  double pair_launch_ms;     /* VS_TIMING_KERNEL: sum of the pair kernel's launch intervals (first warp start to
                                last warp end, device globaltimer; concurrent launches overlap) */
  uint64_t pair_timed_launches;
  double pair_warp_ms;       /* VS_TIMING_KERNEL: sum over every pair-kernel warp of its duration (warp-ms): divided by
                                the busy time and the SM count, the average number of resident pair-kernel warps */
} vs_stats;

/* Instrumentation flags of vs_set_timing (OR-ed):
 *   VS_TIMING_EVENTS  CUDA events around every scoring call of direct (un-graphed) launches -> score_ms;
 *   VS_TIMING_KERNEL  the pair kernel records its launch interval (first warp start, last warp end) on the
 *                     device globaltimer, also inside replayed CUDA graphs -> pair_busy_ms, pair_launch_ms;
 *   VS_TIMING_CENSUS  pair-kernel launches count the pairs within rc (another instantiation of the same
 *                     arithmetic: scores are bitwise unchanged) -> pairs_within.
 * Changing the flags selects another CUDA graph of vs_run. */
#define VS_TIMING_EVENTS 1
#define VS_TIMING_KERNEL 2
#define VS_TIMING_CENSUS 4
VS_API vs_status vs_set_timing(vs_ctx* c, int flags);
/* Synchronises the ctx's device and returns counters since the last reset. */
VS_API vs_status vs_get_stats(vs_ctx* c, vs_stats* out);
VS_API vs_status vs_reset_stats(vs_ctx* c);
/* VS_TIMING_KERNEL: the pair kernel's launch intervals since the last reset as (start, end) device globaltimer ns
 * pairs into out[cap][2] (one clock per device, so the intervals of several contexts can be merged: their union is
 * the time some pair kernel ran).  Returns the number recorded (only min(n, cap) written; cap 0 with out NULL
 * queries n), 0 if kernel timing was never enabled, -1 on error (vs_last_error). */
VS_API int64_t vs_pair_intervals(vs_ctx* c, uint64_t* out, int64_t cap);
/* Per-spot receptor list lengths (cutoff mode) or n_rec (all pairs). */
VS_API vs_status vs_list_lengths(vs_ctx* c, int32_t* out /*[n_spots]*/);

/* ---- debug / lockstep trace -------------------------------------------- */
typedef enum {
  VS_TRACE_INIT = 0,      /* S after Initialize's generation, before scoring (score field 0) */
  VS_TRACE_SCORED = 1,    /* population after scoring (S at g = 0, Scom at g >= 1) */
  VS_TRACE_SELECT = 2,    /* J: indices of the elements Improve works on (idx only) */
  VS_TRACE_LS = 3,        /* population after local-search step l */
  VS_TRACE_SORTED = 4,    /* S after the generation-0 sort */
  VS_TRACE_COMBINED = 5,  /* Scom after Select + Combine, before scoring */
  VS_TRACE_INCLUDED = 6   /* S after Include at generation g */
} vs_trace_stage;

/* poses8 [n_sel][count][8] = (w,x,y,z,tx,ty,tz,score) or NULL;
 * idx [n_sel][count] or NULL.  Host memory valid during the call only. */
typedef void (*vs_trace_fn)(void* user, int32_t stage, int32_t g, int32_t l, int32_t n_sel, int32_t count,
                            const float* poses8, const int32_t* idx);

/* vs_run with a callback after every stage (synchronises at each stage). */
VS_API vs_status vs_run_trace(vs_ctx* c, const vs_mh_params* mp, uint64_t seed, int32_t n_sel, const int32_t* spot_ids,
                       float* best_pose_out, float* best_score_out, vs_trace_fn fn, void* user);

/* Device Philox4x32-10 for n counters: ctr [n][4], key [2] -> out [n][4]
 * (host buffers; for known-answer tests of the device generator). */
VS_API vs_status vs_debug_philox(int64_t n, const uint32_t* ctr, const uint32_t* key, uint32_t* out);

#ifdef __cplusplus
}
#endif
#endif /* VS_H */
