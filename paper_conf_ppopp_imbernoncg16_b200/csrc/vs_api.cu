// vs_api.cu -- C ABI (include/vs.h): context, validation, list building and the
// device-resident generation loop of Algorithm 1.
//
// The paper's host loop copies the candidate set to each GPU and back for
// every scoring call (Algorithm 2).  Here the whole population
// lives in HBM for the run; the host only sequences kernel launches (spot
// groups on up to 12 streams, captured as one CUDA graph on repeated calls),
// and the device boundary is crossed at the start (seed, spot ids) and the
// end (best pose + score per spot).
#include <algorithm>
#include <chrono>
#include <cmath>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <mutex>
#include <unordered_map>
#include <new>
#include <string>
#include <vector>

#include "../../include/vs.h"
#include "vs_kernels.cuh"

using namespace vsk;

namespace {

thread_local std::string g_err;

vs_status set_err(vs_status s, const std::string& msg) {
  g_err = msg;
  return s;
}

// built-in atom types (R4/R5): C N O S H HD X
const float kSigma[7] = {3.400f, 3.250f, 2.960f, 3.564f, 2.650f, 1.069f, 0.0f};
const float kEps[7] = {0.1094f, 0.170f, 0.210f, 0.250f, 0.0157f, 0.0157f, 0.0f};
const int kRole[7] = {0, 2, 2, 0, 0, 1, 0};

struct DeviceGuard {
  int prev = -1;
  explicit DeviceGuard(int dev) {
    if (cudaGetDevice(&prev) != cudaSuccess) prev = -1;
    if (prev != dev) cudaSetDevice(dev);
  }
  ~DeviceGuard() {
    int cur;
    if (prev >= 0 && cudaGetDevice(&cur) == cudaSuccess && cur != prev) cudaSetDevice(prev);
  }
};

// ---------------------------------------------------------------- device memory cache
// A context allocates ~20 device buffers at vs_create / first vs_run and frees them at vs_destroy; on the B200 box
// cudaMalloc / cudaFree cost 1-30 ms each, erratically (measured inside vs_destroy with VS_DEBUG_TIMING), which
// dominated the end-to-end time of short runs and of the one-context-per-ligand sweep.  Freed blocks are kept per
// device and handed to later allocations of the same bucket (size rounded up to a power of two below 2 MiB, to a
// 2 MiB multiple above).  Cached free bytes per device are capped (VS_POOL_CACHE_MB, default 8192); beyond that,
// and for pointers the cache did not allocate, frees go to the driver.  A block is returned only when no GPU work
// can still use it: every caller synchronises first (vs_destroy, DevBuf regrow, the end of vs_create).
namespace pool {
struct Dev {
  std::unordered_map<size_t, std::vector<void*>> free;
  std::unordered_map<void*, size_t> live;
  size_t cached = 0;
};
std::mutex mu;
std::unordered_map<int, Dev>& devs() {
  static auto* d = new std::unordered_map<int, Dev>();  // never destroyed: frees may run during process teardown
  return *d;
}
size_t bucket(size_t b) {
  constexpr size_t big = size_t(2) << 20;
  if (b <= big) {
    size_t k = 512;
    while (k < b) k <<= 1;
    return k;
  }
  return (b + big - 1) / big * big;
}
size_t cache_cap() {
  static const size_t cap = [] {
    const char* v = std::getenv("VS_POOL_CACHE_MB");
    return (size_t)(v ? std::strtoull(v, nullptr, 10) : 8192ull) << 20;
  }();
  return cap;
}
void trim(int dev) {  // hand every cached block of dev back to the driver
  std::vector<void*> ps;
  {
    std::lock_guard<std::mutex> g(mu);
    Dev& d = devs()[dev];
    for (auto& kv : d.free)
      for (void* q : kv.second) ps.push_back(q);
    d.free.clear();
    d.cached = 0;
  }
  for (void* q : ps) cudaFree(q);
}
cudaError_t alloc(void** p, size_t bytes) {
  *p = nullptr;
  int dev = 0;
  cudaGetDevice(&dev);
  const size_t b = bucket(std::max<size_t>(bytes, 1));
  {
    std::lock_guard<std::mutex> g(mu);
    Dev& d = devs()[dev];
    auto it = d.free.find(b);
    if (it != d.free.end() && !it->second.empty()) {
      *p = it->second.back();
      it->second.pop_back();
      d.cached -= b;
      d.live[*p] = b;
      return cudaSuccess;
    }
  }
  cudaError_t e = cudaMalloc(p, b);
  if (e == cudaErrorMemoryAllocation) {  // cached blocks of other sizes may be what is missing
    cudaGetLastError();
    trim(dev);
    e = cudaMalloc(p, b);
  }
  if (e != cudaSuccess) {
    *p = nullptr;
    return e;
  }
  std::lock_guard<std::mutex> g(mu);
  devs()[dev].live[*p] = b;
  return cudaSuccess;
}
template <typename T>
cudaError_t alloc(T** p, size_t bytes) {
  void* q = nullptr;
  const cudaError_t e = alloc(&q, bytes);
  *p = static_cast<T*>(q);
  return e;
}
void release(void* p) {
  if (!p) return;
  int dev = 0;
  cudaGetDevice(&dev);
  {
    std::lock_guard<std::mutex> g(mu);
    Dev& d = devs()[dev];
    auto it = d.live.find(p);
    if (it != d.live.end()) {
      const size_t b = it->second;
      d.live.erase(it);
      if (d.cached + b <= cache_cap()) {
        d.free[b].push_back(p);
        d.cached += b;
        return;
      }
    }
  }
  cudaFree(p);
}
}  // namespace pool

struct DevBuf {
  void* p = nullptr;
  size_t cap = 0;
  cudaError_t ensure(size_t bytes) {
    if (bytes <= cap) return cudaSuccess;
    if (p) {
      cudaDeviceSynchronize();  // earlier launches may still read the old block
      pool::release(p);
    }
    p = nullptr;
    cap = 0;
    cudaError_t e = pool::alloc(&p, bytes);
    if (e == cudaSuccess) cap = bytes;
    return e;
  }
  void release() {
    pool::release(p);
    p = nullptr;
    cap = 0;
  }
};

#ifndef VS_NSUB
#define VS_NSUB 12
#endif
constexpr int NSUB = VS_NSUB;  // spot groups (streams) of one vs_run
// cells per axis of the per-spot list grid: 18 for contexts with 1 or 2 list splits (throughput-bound runs: fewer,
// longer row runs), 20 with 4 splits (latency-bound runs: each split warp streams fewer atoms).  Medium, ms: S 1,
// 500 spots: G 24 / 20 / 18 / 16 / 14 / 12 465.3 / 464.2 / 458.9 / 460.3 / 460.1 / 462.4; S 2, 125 spots G 24 / 20 /
// 18 / 16 / 14: 129.0 / 128.1 / 127.0 / 127.4 / 133.5; S 4, 63 spots G 24 / 20 / 16: 78.0 / 77.1 / 78.5; small (S 4)
// 17.9 / 17.57 / 18.2; large 500 spots (S 1) G 24 / 20 / 18 / 16: 1260 / 1256 / 1248 / 1250 (profiles/r02_notes.md).
// S must divide G (the pair kernel assigns cell rows to splits by cy mod S).
int cell_grid(int nsplit) {
  const int g = VS_CELL_G > 0 ? VS_CELL_G : (nsplit >= 4 ? 20 : 18);
  return g;
}
static_assert(vsk::CELL_GMAX % vsk::CELL_NSPLIT == 0 && 20 % vsk::CELL_NSPLIT == 0 && 18 % 2 == 0,
              "the pair kernel assigns cell rows to splits by cy mod S (18: 1 or 2 splits, 20: 4)");
static_assert(VS_CELL_G <= vsk::CELL_GMAX && VS_CELL_G % vsk::CELL_NSPLIT == 0, "VS_CELL_G");
#ifndef VS_GROUP_SPOTS
#define VS_GROUP_SPOTS 8    // spots per stream group at least
#endif
#ifndef VS_BIG_RUN_SPOTS
#define VS_BIG_RUN_SPOTS 256  // runs of at least this many spots use at most VS_BIG_RUN_GROUPS streams
#endif
#ifndef VS_BIG_RUN_GROUPS
#define VS_BIG_RUN_GROUPS 12
#endif
#ifndef VS_FILL_WARPS
#define VS_FILL_WARPS 4096    // pair-kernel warps below which a scoring round uses KP = 1 chunks (launch shape); 2048 -> 4096:
                              // medium 32 spots (S 4) 56.0 -> 52.2 ms, 125 spots (S 1) 150.4 -> 133.1, others unchanged
#endif
#ifndef VS_TRIGGER_SPOTS
#define VS_TRIGGER_SPOTS 0    // runs of at most this many spots: PDL early trigger (latency-bound)
#endif
#ifndef VS_DIRECT_GROUP_SPOTS
#define VS_DIRECT_GROUP_SPOTS 16  // un-graphed runs: spots per stream group at least (small e2e 34 -> 24 ms / step)
#endif
#ifndef VS_GRAPH_CACHE
#define VS_GRAPH_CACHE 4      // CUDA graphs kept per context
#endif
#ifndef VS_KT_CAP
#define VS_KT_CAP (1 << 20)   // pair-kernel launch intervals kept (instrumentation)
#endif

enum Buf { B_SEG, B_SA, B_SB, B_C, B_J, B_SPOT, B_Q, B_T, B_OUT, B_VALID, B_COUNTS, B_PP, B_BP, B_CUR,
           B_SORTED, B_ORIG, B_BEST, B_BESTS, B_PBUF, B_ITEMS, B_E, B_COUNT };

bool finite_arr(const float* p, int64_t n) {
  for (int64_t i = 0; i < n; ++i)
    if (!std::isfinite(p[i])) return false;
  return true;
}

}  // namespace

struct vs_ctx {
  int dev = 0;
  int n_rec = 0, n_lig = 0, n_spots = 0;
  bool all_pairs = false;
  int dielectric = 0;
  float T = 3.0f, rc = 0.0f, rc2 = INFINITY, inv_rc2 = 0.0f, r2min = 0.01f, hbC = 0.0f, hbD = 0.0f;
  int n_sm = 148;
  std::vector<int> h_list_len;
  int64_t list_total = 0;
  RecAtom* d_lists = nullptr;
  int* d_list_off = nullptr;
  int* d_list_len = nullptr;
  float4* d_shift = nullptr;
  int* d_iota = nullptr;
  unsigned long long* d_counters = nullptr;  // [0] pairs evaluated, [1] poses, [2] workload pairs, [3] within rc
  // vs_run's scored poses and workload pairs, counted on the host from the run's parameters (K3 counts them on the
  // device only for vs_score_poses: a burst of same-address atomics from every K3 CTA cost 0.4 % of a medium step)
  unsigned long long host_poses = 0, host_pairs = 0;
  uint64_t* d_seed = nullptr;           // seed of the current run (device copy)
  uint16_t* d_cells = nullptr;          // cutoff mode: [n_spots][cg^3 + 1] cell starts of the cell-sorted lists
  int cell_g = 18;                      // cells per axis of the list grid (cell_grid)
  float cR = 0.0f, ch = 0.0f, cinv_h = 0.0f;
  long long fill_warps = VS_FILL_WARPS;  // launch shape target (speed only)
  int nsplit = 1;                        // canonical receptor-list splits (vs_score_params.list_splits)
  int force_kp = 0;                      // VS_SHAPE=kp (experiments)
  int direct_group_spots = VS_DIRECT_GROUP_SPOTS;  // spots per stream group at least, un-graphed runs
  int trigger_spots = VS_TRIGGER_SPOTS;            // runs of at most this many spots use the PDL early trigger
  float4* d_ligx = nullptr;             // [n_lig] centred local coordinates, w = class
  float4* d_ligp = nullptr;             // [n_lig] es, c12, c6, donor
  int* d_lig_rank = nullptr;            // [n_lig] rank within the class
  int nn = 0, nh = 0, H2 = 0, H1 = 0;  // H-bond slot pairs of the KP = 2 / KP = 1 pair kernels
  float W = 0.0f, inv_hm = 0.0f;
  cudaStream_t stream = nullptr;
  cudaStream_t sub[NSUB] = {};          // per-spot-group streams of vs_run
  cudaEvent_t ev_fork = nullptr, ev_join[NSUB] = {};
  cudaEvent_t ev_in = nullptr, ev_out = nullptr;  // caller stream <-> ctx stream ordering of the async entry points
  DevBuf buf[B_COUNT];
  bool poisoned = false;
  // instrumentation
  uint64_t launches = 0, score_launches = 0;
  bool timing = false, ktime = false, census = false;
  unsigned long long* d_kt = nullptr;       // [VS_KT_CAP][KT_WORDS] pair-kernel launch intervals (~start, end, warp ns)
  unsigned long long* d_kt_base = nullptr;  // first slot of the next run's region
  int kt_local = 0;                         // slots used by the run being enqueued
  std::vector<cudaEvent_t> ev;  // pairs (start, end)
  size_t ev_used = 0;
  double score_ms_acc = 0.0;
  uint64_t timed_acc = 0;
  // CUDA graphs of vs_run: captured on the second identical call, a few kept (LRU) so that runs of a few shapes
  // (spot-chunk sizes of a multi-GPU queue) all replay
  struct Graph {
    unsigned char key[256];
    cudaGraphExec_t exec = nullptr;
    uint64_t launches = 0, score_launches = 0, used = 0;
  };
  bool graphs = true, capturing = false, has_last = false;
  std::vector<Graph> gcache;
  uint64_t gclock = 0;
  unsigned char last_key[256] = {};
};

namespace {

// A failed allocation leaves the ctx usable (VS_ERR_OUT_OF_MEMORY); any other CUDA error poisons it.
vs_status cuda_fail(vs_ctx* c, cudaError_t e, const char* where) {
  const bool oom = e == cudaErrorMemoryAllocation;
  if (oom) cudaGetLastError();  // reset the (non-sticky) last-error state
  if (c && !oom) c->poisoned = true;
  return set_err(oom ? VS_ERR_OUT_OF_MEMORY : VS_ERR_CUDA, std::string(where) + ": " + cudaGetErrorString(e));
}

#define CK(expr, where)                                 \
  do {                                                  \
    cudaError_t e_ = (expr);                            \
    if (e_ != cudaSuccess) return cuda_fail(c, e_, where); \
  } while (0)

vs_status check_mh(const vs_mh_params* mp) {
  if (!mp) return set_err(VS_ERR_INVALID_ARGUMENT, "mh params: NULL");
  if (mp->population < 1 || mp->population > 2048) return set_err(VS_ERR_INVALID_ARGUMENT, "population must be in [1, 2048]");
  if (mp->generations < 0) return set_err(VS_ERR_INVALID_ARGUMENT, "generations must be >= 0");
  if (mp->generations > 0 && mp->population < 2)
    return set_err(VS_ERR_INVALID_ARGUMENT, "population must be >= 2 when generations > 0");
  if (mp->ls_steps < 0) return set_err(VS_ERR_INVALID_ARGUMENT, "ls_steps must be >= 0");
  if (mp->ls_neighbours < 1 || mp->ls_neighbours > 64)
    return set_err(VS_ERR_INVALID_ARGUMENT, "ls_neighbours must be in [1, 64]");
  // the LS Philox counter word is (TAG_LS << 24) | (2 (l K + k) + 1): it must stay below 2^24 (R23)
  if ((long long)mp->ls_steps * mp->ls_neighbours > (1ll << 23))
    return set_err(VS_ERR_INVALID_ARGUMENT, "ls_steps x ls_neighbours must be <= 2^23");
  if (!(mp->improve_frac >= 0.0f && mp->improve_frac <= 1.0f)) return set_err(VS_ERR_INVALID_ARGUMENT, "improve_frac must be in [0, 1]");
  if (!(mp->p_mut >= 0.0f && mp->p_mut <= 1.0f)) return set_err(VS_ERR_INVALID_ARGUMENT, "p_mut must be in [0, 1]");
  const float st[4] = {mp->mut_trans, mp->mut_rot, mp->ls_trans, mp->ls_rot};
  for (float v : st)
    if (!(std::isfinite(v) && v >= 0.0f)) return set_err(VS_ERR_INVALID_ARGUMENT, "step sizes must be finite and >= 0");
  return VS_OK;
}

// m = clamp(round-half-up(f * P), 1, P) with f the fp32 ABI value (R17)
int improve_count(const vs_mh_params* mp) {
  long long m = std::llround((double)mp->improve_frac * (double)mp->population);
  if (m < 1) m = 1;
  if (m > mp->population) m = mp->population;
  return (int)m;
}

vs_status collect_timing(vs_ctx* c) {
  for (size_t i = 0; i + 1 < c->ev_used; i += 2) {
    float ms = 0.0f;
    CK(cudaEventSynchronize(c->ev[i + 1]), "cudaEventSynchronize");
    CK(cudaEventElapsedTime(&ms, c->ev[i], c->ev[i + 1]), "cudaEventElapsedTime");
    c->score_ms_acc += ms;
    c->timed_acc++;
  }
  c->ev_used = 0;
  return VS_OK;
}

// Launch shape of a scoring launch: KP packed item pairs per lane (items per chunk = 64 KP); every chunk takes one
// warp per canonical list split (S, a context property).  KP changes only how the items are cut into warps --
// never a result (vs_cells.cu header) -- so it is chosen per launch for speed: KP 2 unless the run's scoring round
// (all its spots) would have fewer than fill_warps warps, then KP 1 (twice the warps, each with half the items) for
// latency-bound launches (few spots, Improve's m poses per spot).  (A warp looping over several splits was
// measured slower than one warp per split even for latency-bound launches: profiles/r02_notes.md.)
struct Shape {
  int kp, H, cn, chb, w, S;
  int nn, nh, merged;  // item classes of the launch (merged: every atom in the H-bond class, one curve order)
  int nsg() const { return S; }
};
Shape shape_of(const vs_ctx* c, int kp, int w) {
  Shape s;
  s.S = c->nsplit;
  s.kp = kp;
  s.H = kp == 2 ? c->H2 : c->H1;
  s.cn = 64 * kp;
  s.chb = 64 * s.H;
  s.w = w;
  s.nn = c->nn;
  s.nh = c->nh;
  s.merged = 0;
  // a KP = 1 chunk has one slot pair, an H-bond pair whenever the ligand has H-bond atoms: its items then go in one
  // class and one curve order (spatially tighter chunks at no extra cost per pair; layout only, never a result)
  if (kp == 1 && s.H == 1 && c->nn > 0) {
    s.nn = 0;
    s.nh = c->n_lig;
    s.merged = 1;
  }
  return s;
}
Shape choose_shape(const vs_ctx* c, long long n_seg, int seg_n) {
  if (c->force_kp) return shape_of(c, c->force_kp, 1);
  const Shape s2 = shape_of(c, 2, 1);
  if (n_seg * cell_chunks(seg_n, s2.nn, s2.nh, s2.cn, s2.chb) * s2.nsg() >= c->fill_warps) return s2;
  return shape_of(c, 1, 1);
}
void apply_shape(CellArgs& a, const Shape& s) {
  a.kp = s.kp;
  a.H = s.H;
  a.cn = s.cn;
  a.chb = s.chb;
  a.w = s.w;
  a.nsplit = s.S;
  a.nn = s.nn;
  a.nh = s.nh;
  a.merged = s.merged;
}

CellArgs cell_base(vs_ctx* c) {
  CellArgs a;
  std::memset(&a, 0, sizeof(a));
  a.lists = c->d_lists;
  a.list_off = c->d_list_off;
  a.list_len = c->d_list_len;
  a.cells = c->all_pairs ? nullptr : c->d_cells;
  a.cR = c->cR;
  a.ch = c->ch;
  a.cinv_h = c->cinv_h;
  a.cg = c->cell_g;
  a.ligx = c->d_ligx;
  a.ligp = c->d_ligp;
  a.lig_rank = c->d_lig_rank;
  a.n_lig = c->n_lig;
  apply_shape(a, shape_of(c, 2, 4));
  a.shift = c->d_shift;
  a.W = c->W;
  a.inv_hm = c->inv_hm;
  a.cut = c->all_pairs ? 0 : 1;
  a.K = 1;
  a.r2min = c->r2min;
  a.rc = c->rc;
  a.rc2 = c->rc2;
  a.inv_rc2 = c->inv_rc2;
  a.hbC = c->hbC;
  a.hbD = c->hbD;
  a.T = c->T;
  a.counters = c->d_counters;
  a.census = c->census ? 1 : 0;
  a.kt = c->ktime ? c->d_kt : nullptr;
  a.kt_base = c->d_kt_base;
  a.kt_cap = VS_KT_CAP;
  a.seedp = c->d_seed;
  return a;
}

vs_status cell_launch(vs_ctx* c, const CellArgs& a_in, long long n_poses, int nb2, cudaStream_t st) {
  CellArgs a = a_in;
  if (a.kt) a.kt_slot = c->kt_local++;
  cudaEvent_t e0 = nullptr, e1 = nullptr;
  const bool timed = c->timing && !c->capturing;
  if (timed) {
    if (c->ev_used + 2 > c->ev.size()) {
      for (int i = 0; i < 64; ++i) {
        cudaEvent_t e;
        CK(cudaEventCreate(&e), "cudaEventCreate");
        c->ev.push_back(e);
      }
    }
    e0 = c->ev[c->ev_used];
    e1 = c->ev[c->ev_used + 1];
    c->ev_used += 2;
    CK(cudaEventRecord(e0, st), "cudaEventRecord");
  }
  CK(launch_cell_score(a, c->dielectric, n_poses, nb2, st), "cells score launch");
  c->launches += 3;
  c->score_launches++;
  if (timed) CK(cudaEventRecord(e1, st), "cudaEventRecord");
  return VS_OK;
}

struct Tracer {
  vs_trace_fn fn = nullptr;
  void* user = nullptr;
  std::vector<float> hp;
  std::vector<int32_t> hi;
};

vs_status trace_poses(vs_ctx* c, Tracer* tr, cudaStream_t st, int stage, int g, int l, int n_sel, int count,
                      const PoseRec* d) {
  if (!tr || !tr->fn) return VS_OK;
  tr->hp.resize((size_t)n_sel * count * 8);
  CK(cudaMemcpyAsync(tr->hp.data(), d, tr->hp.size() * sizeof(float), cudaMemcpyDeviceToHost, st), "trace D2H");
  CK(cudaStreamSynchronize(st), "trace sync");
  tr->fn(tr->user, stage, g, l, n_sel, count, tr->hp.data(), nullptr);
  return VS_OK;
}

vs_status trace_idx(vs_ctx* c, Tracer* tr, cudaStream_t st, int stage, int g, int n_sel, int count, const int* d) {
  if (!tr || !tr->fn) return VS_OK;
  tr->hi.resize((size_t)n_sel * count);
  CK(cudaMemcpyAsync(tr->hi.data(), d, tr->hi.size() * sizeof(int32_t), cudaMemcpyDeviceToHost, st), "trace D2H");
  CK(cudaStreamSynchronize(st), "trace sync");
  tr->fn(tr->user, stage, g, 0, n_sel, count, nullptr, tr->hi.data());
  return VS_OK;
}

// Everything one run's enqueued work depends on except the seed (also the CUDA-graph cache key).
struct Body {
  vs_mh_params mp;
  int m, ns;
  int* seg;
  PoseRec *SA, *SB, *CC;
  int* JJ;
  float *best_pose, *best_score;
  // scoring scratch
  PoseRec* pbuf;
  float4* items;
  double* E;
  int emax;  // E entries per spot and ligand atom: max over the launches of (poses per spot x split groups)
  int census, ktime;  // instrumentation (a different pair-kernel instantiation / extra arguments)
};

static_assert(sizeof(Body) <= 256, "graph key storage");

// One group of spots running Algorithm 1 on its own stream.
struct Group {
  int ns = 0;
  const int* seg = nullptr;
  PoseRec *S = nullptr, *S2 = nullptr, *C = nullptr;
  int* J = nullptr;
  cudaStream_t st = nullptr;
  CellArgs cplain, cls;                // scoring launches: plain (a whole population) and Improve (LS)
  int cplain_blocks = 0, cls_blocks = 0;
  bool in_b = false;  // the current population S sits in the second (B) buffer
  int trig = 0;       // PDL early trigger for the group's chain (latency-bound runs)
};

// Improve (R16-R17): the best m of X by (score, index), then L fused
// perturb -> score -> accept launches.
vs_status improve_step(vs_ctx* c, Group& q, const vs_mh_params* mp, int m, PoseRec* X, int g, Tracer* tr) {
  const int P = mp->population;
  CK(launch_popsort(0, X, nullptr, nullptr, q.J, q.ns, P, m, q.trig, q.st), "select launch");
  c->launches++;
  vs_status r = trace_idx(c, tr, q.st, VS_TRACE_SELECT, g, q.ns, m, q.J);
  if (r != VS_OK) return r;
  for (int l = 0; l < mp->ls_steps; ++l) {
    CellArgs a = q.cls;
    a.poses = X;
    a.g = g;
    a.l = l;
    if ((r = cell_launch(c, a, (long long)q.ns * a.seg_size, q.cls_blocks, q.st)) != VS_OK) return r;
    if ((r = trace_poses(c, tr, q.st, VS_TRACE_LS, g, l, q.ns, P, X)) != VS_OK) return r;
  }
  return VS_OK;
}

// Initialize(S): random population, scored, improved when f > 0, sorted.
vs_status gen_initialize(vs_ctx* c, Group& q, const vs_mh_params* mp, int m, Tracer* tr) {
  const int P = mp->population;
  CK(launch_init(q.S, q.ns, P, q.seg, c->d_seed, c->T, q.trig, q.st), "init launch");
  c->launches++;
  vs_status r = trace_poses(c, tr, q.st, VS_TRACE_INIT, 0, 0, q.ns, P, q.S);
  if (r != VS_OK) return r;
  {
    CellArgs a = q.cplain;
    a.poses = q.S;
    if ((r = cell_launch(c, a, (long long)q.ns * P, q.cplain_blocks, q.st)) != VS_OK) return r;
  }
  if ((r = trace_poses(c, tr, q.st, VS_TRACE_SCORED, 0, 0, q.ns, P, q.S)) != VS_OK) return r;
  if (mp->improve_frac > 0.0f && (r = improve_step(c, q, mp, m, q.S, 0, tr)) != VS_OK) return r;
  CK(launch_popsort(1, q.S, nullptr, q.S2, nullptr, q.ns, P, m, q.trig, q.st), "sort launch");
  c->launches++;
  std::swap(q.S, q.S2);
  q.in_b = !q.in_b;
  return trace_poses(c, tr, q.st, VS_TRACE_SORTED, 0, 0, q.ns, P, q.S);
}

// One pass of the while-loop body: Select + Combine, score, Improve, Include.
vs_status gen_step(vs_ctx* c, Group& q, const vs_mh_params* mp, int m, int g, Tracer* tr) {
  const int P = mp->population;
  CK(launch_combine(q.S, q.C, q.ns, P, q.seg, c->d_seed, g, mp->p_mut, mp->mut_trans, mp->mut_rot, c->T, q.trig, q.st),
     "combine launch");
  c->launches++;
  vs_status r = trace_poses(c, tr, q.st, VS_TRACE_COMBINED, g, 0, q.ns, P, q.C);
  if (r != VS_OK) return r;
  {
    CellArgs a = q.cplain;
    a.poses = q.C;
    if ((r = cell_launch(c, a, (long long)q.ns * P, q.cplain_blocks, q.st)) != VS_OK) return r;
  }
  if ((r = trace_poses(c, tr, q.st, VS_TRACE_SCORED, g, 0, q.ns, P, q.C)) != VS_OK) return r;
  if (mp->improve_frac > 0.0f && (r = improve_step(c, q, mp, m, q.C, g, tr)) != VS_OK) return r;
  CK(launch_popsort(2, q.S, q.C, q.S2, nullptr, q.ns, P, m, q.trig, q.st), "include launch");
  c->launches++;
  std::swap(q.S, q.S2);
  q.in_b = !q.in_b;
  return trace_poses(c, tr, q.st, VS_TRACE_INCLUDED, g, 0, q.ns, P, q.S);
}

// Everything a run enqueues after its inputs are on the device (the part a CUDA graph captures).
vs_status enqueue_body(vs_ctx* c, const Body& b, cudaStream_t st, Tracer* tr) {
  const vs_mh_params* mp = &b.mp;
  const int P = mp->population, m = b.m, ns = b.ns;
  c->kt_local = 0;
  // Spots are independent: split them into groups whose generation loops run on separate
  // streams, enqueued generation by generation, so one group's kernels fill the wave tails of
  // another's.
  // Stream count (measured on B200, profiles/r01_notes.md): runs are chains of partly latency-bound launches and
  // gain from extra streams (64 spots: 4 -> 8 streams, 25.8 -> 24.6 ms / step; 500 spots: 8 -> 12 streams, with
  // the pair kernel at 20 CTAs / SM, 564 -> 553 ms / step), but every stream adds launches to a context's first,
  // un-graphed run (host-bound: 16 streams doubled it on the small config), hence >= 8 spots per group.
  int G = std::max(1, std::min(NSUB, ns / VS_GROUP_SPOTS));
  if (ns >= VS_BIG_RUN_SPOTS) G = std::min(G, VS_BIG_RUN_GROUPS);
  // a run enqueued launch by launch (not captured into a graph: a context's first call) is bound by the host's
  // launch rate when it has few spots per group: fewer groups, fewer launches (results do not depend on grouping)
  if (!c->capturing) G = std::max(1, std::min(G, ns / c->direct_group_spots));
  if (tr) G = 1;
  Group grp[NSUB];
  CK(cudaEventRecord(c->ev_fork, st), "event record");
  for (int gi = 0; gi < G; ++gi) {
    const int k0 = (int)((int64_t)ns * gi / G), k1 = (int)((int64_t)ns * (gi + 1) / G);
    Group& q = grp[gi];
    q.ns = k1 - k0;
    q.seg = b.seg + k0;
    q.S = b.SA + (size_t)k0 * P;
    q.S2 = b.SB + (size_t)k0 * P;
    q.C = b.CC + (size_t)k0 * P;
    q.J = b.JJ + (size_t)k0 * m;
    q.st = G > 1 ? c->sub[gi] : st;
    if (G > 1) CK(cudaStreamWaitEvent(q.st, c->ev_fork, 0), "stream wait");
    {
      const int mk = m * mp->ls_neighbours, maxpose = std::max(P, mk);
      const Shape shp = choose_shape(c, ns, P), shl = choose_shape(c, ns, mk);  // shapes from the whole run's size
      CellArgs& cp = q.cplain;
      cp = cell_base(c);
      apply_shape(cp, shp);
      cp.nseg = q.ns;
      cp.seg_spot = q.seg;
      cp.uniform = 1;
      cp.seg_size = P;
      cp.seg_stride = P;
      cp.P = P;
      cp.mode = MODE_PLAIN;
      cp.nch_u = cell_chunks(P, shp.nn, shp.nh, shp.cn, shp.chb);
      cp.pbuf = b.pbuf + (size_t)k0 * maxpose;
      cp.items = b.items + (size_t)k0 * maxpose * c->n_lig;
      cp.E = b.E + (size_t)k0 * c->n_lig * b.emax;
      cp.E_stride = (long long)q.ns * P * c->n_lig;
      CellArgs& cl = q.cls;
      cl = cp;
      apply_shape(cl, shl);
      cl.mode = MODE_LS;
      cl.seg_size = mk;
      cl.nch_u = cell_chunks(mk, shl.nn, shl.nh, shl.cn, shl.chb);
      cl.E_stride = (long long)q.ns * mk * c->n_lig;
      cl.J = q.J;
      cl.m = m;
      cl.K = mp->ls_neighbours;
      cl.ls_trans = mp->ls_trans;
      cl.ls_rot = mp->ls_rot;
      // latency-bound runs (few spots): every chain kernel triggers its successor's launch at entry
      q.trig = ns <= c->trigger_spots ? 1 : 0;
      cp.trig = cl.trig = q.trig;
      q.cplain_blocks = q.ns * cp.nch_u * shp.nsg();
      q.cls_blocks = q.ns * cl.nch_u * shl.nsg();
    }
  }
  vs_status r;
  for (int gi = 0; gi < G; ++gi)
    if ((r = gen_initialize(c, grp[gi], mp, m, tr)) != VS_OK) return r;
  for (int g = 1; g <= mp->generations; ++g)         // End(S): fixed G (R20)
    for (int gi = 0; gi < G; ++gi)
      if ((r = gen_step(c, grp[gi], mp, m, g, tr)) != VS_OK) return r;
  if (G > 1)
    for (int gi = 0; gi < G; ++gi) {
      CK(cudaEventRecord(c->ev_join[gi], grp[gi].st), "event record");
      CK(cudaStreamWaitEvent(st, c->ev_join[gi], 0), "stream wait");
    }
  CK(launch_best(grp[0].in_b ? b.SB : b.SA, ns, P, b.best_pose, b.best_score, st), "best launch");
  c->launches++;
  if (b.ktime) {
    CK(launch_kt_advance(c->d_kt_base, c->kt_local, st), "kt launch");
    c->launches++;
  }
  return VS_OK;
}

// The generation loop (Algorithm 1) for n_sel spots, all on stream st.
vs_status run_impl(vs_ctx* c, const vs_mh_params* mp, uint64_t seed, int32_t n_sel, const int32_t* spot_ids,
                   float* d_best_pose, float* d_best_score, cudaStream_t st, Tracer* tr) {
  vs_status s = check_mh(mp);
  if (s != VS_OK) return s;
  if (n_sel < 0) return set_err(VS_ERR_INVALID_ARGUMENT, "n_sel must be >= 0");
  if (!spot_ids && n_sel != 0 && n_sel != c->n_spots)
    return set_err(VS_ERR_INVALID_ARGUMENT, "n_sel must be 0 or n_spots when spot_ids is NULL");
  if (spot_ids && n_sel == 0) return set_err(VS_ERR_INVALID_ARGUMENT, "n_sel must be >= 1 with spot_ids");
  const int ns = spot_ids ? n_sel : c->n_spots;
  if (spot_ids)
    for (int k = 0; k < ns; ++k)
      if (spot_ids[k] < 0 || spot_ids[k] >= c->n_spots) return set_err(VS_ERR_INVALID_ARGUMENT, "spot id out of range");
  const int P = mp->population;
  const int m = improve_count(mp);
  const size_t pop_bytes = sizeof(PoseRec) * (size_t)ns * P;
  CK(c->buf[B_SEG].ensure(sizeof(int) * ns), "alloc");
  CK(c->buf[B_SA].ensure(pop_bytes), "alloc");
  CK(c->buf[B_SB].ensure(pop_bytes), "alloc");
  CK(c->buf[B_C].ensure(pop_bytes), "alloc");
  CK(c->buf[B_J].ensure(sizeof(int) * (size_t)ns * m), "alloc");
  int emax = 0;
  {
    const int mk = m * mp->ls_neighbours, maxpose = std::max(P, mk);
    if ((long long)ns * maxpose * c->n_lig >= (1ll << 31))
      return set_err(VS_ERR_INVALID_ARGUMENT, "n_sel x population x n_lig must be < 2^31");
    emax = P * choose_shape(c, ns, P).nsg();
    if (mp->improve_frac > 0.0f) emax = std::max(emax, mk * choose_shape(c, ns, mk).nsg());
    CK(c->buf[B_PBUF].ensure(sizeof(PoseRec) * (size_t)ns * maxpose), "alloc");
    CK(c->buf[B_ITEMS].ensure(sizeof(float4) * (size_t)ns * maxpose * c->n_lig), "alloc");
    CK(c->buf[B_E].ensure(sizeof(double) * (size_t)ns * c->n_lig * emax), "alloc");
  }
  {  // every spot scores (G + 1) x (P + L m K) poses (init / Combine rounds, Improve proposals), n_lig x list pairs each
    const unsigned long long per =
        (unsigned long long)(mp->generations + 1) *
        ((unsigned long long)P + (mp->improve_frac > 0.0f ? (unsigned long long)mp->ls_steps * m * mp->ls_neighbours : 0ull));
    unsigned long long lsum = 0;
    for (int k = 0; k < ns; ++k) lsum += (unsigned long long)c->h_list_len[spot_ids ? spot_ids[k] : k];
    c->host_poses += per * (unsigned long long)ns;
    c->host_pairs += per * (unsigned long long)c->n_lig * lsum;
  }
  int* seg = (int*)c->buf[B_SEG].p;
  if (spot_ids)
    CK(cudaMemcpyAsync(seg, spot_ids, sizeof(int) * ns, cudaMemcpyHostToDevice, st), "H2D spot ids");
  else
    CK(cudaMemcpyAsync(seg, c->d_iota, sizeof(int) * ns, cudaMemcpyDeviceToDevice, st), "D2D spot ids");
  // the seed lives in device memory so that a captured graph can be replayed for any seed
  CK(cudaMemcpyAsync(c->d_seed, &seed, sizeof(uint64_t), cudaMemcpyHostToDevice, st), "H2D seed");
  Body b;
  std::memset(&b, 0, sizeof(b));  // padding bytes take part in the graph-cache key comparison
  b.mp = *mp;
  b.m = m;
  b.ns = ns;
  b.seg = seg;
  b.SA = (PoseRec*)c->buf[B_SA].p;
  b.SB = (PoseRec*)c->buf[B_SB].p;
  b.CC = (PoseRec*)c->buf[B_C].p;
  b.JJ = (int*)c->buf[B_J].p;
  b.best_pose = d_best_pose;
  b.best_score = d_best_score;
  {
    b.pbuf = (PoseRec*)c->buf[B_PBUF].p;
    b.items = (float4*)c->buf[B_ITEMS].p;
    b.E = (double*)c->buf[B_E].p;
    b.emax = emax;
  }
  b.census = c->census ? 1 : 0;
  b.ktime = c->ktime ? 1 : 0;
  if (tr || !c->graphs) return enqueue_body(c, b, st, tr);

  // CUDA graph of the whole run: captured on the second identical call, replayed afterwards
  // (the ~4 + 2 L launches per generation and spot group then cost one graph launch).
  for (auto& gr : c->gcache)
    if (std::memcmp(&b, gr.key, sizeof(Body)) == 0) {
      CK(cudaGraphLaunch(gr.exec, st), "graph launch");
      c->launches += gr.launches;
      c->score_launches += gr.score_launches;
      gr.used = ++c->gclock;
      return VS_OK;
    }
  const bool seen = c->has_last && std::memcmp(&b, &c->last_key, sizeof(Body)) == 0;
  std::memcpy(&c->last_key, &b, sizeof(Body));
  c->has_last = true;
  if (!seen) return enqueue_body(c, b, st, tr);
  if (c->gcache.size() >= VS_GRAPH_CACHE) {  // evict the least recently used graph
    size_t lru = 0;
    for (size_t i = 1; i < c->gcache.size(); ++i)
      if (c->gcache[i].used < c->gcache[lru].used) lru = i;
    cudaGraphExecDestroy(c->gcache[lru].exec);
    c->gcache.erase(c->gcache.begin() + lru);
  }
  const uint64_t l0 = c->launches, s0 = c->score_launches;
  CK(cudaStreamBeginCapture(st, cudaStreamCaptureModeThreadLocal), "begin capture");
  c->capturing = true;
  vs_status r = enqueue_body(c, b, st, tr);
  c->capturing = false;
  cudaGraph_t graph = nullptr;
  cudaError_t e = cudaStreamEndCapture(st, &graph);
  if (r != VS_OK) {
    if (graph) cudaGraphDestroy(graph);
    return r;
  }
  CK(e, "end capture");
  vs_ctx::Graph gr;
  e = cudaGraphInstantiate(&gr.exec, graph, 0);
  cudaGraphDestroy(graph);
  CK(e, "graph instantiate");
  std::memcpy(gr.key, &b, sizeof(Body));
  gr.launches = c->launches - l0;
  gr.score_launches = c->score_launches - s0;
  gr.used = ++c->gclock;
  c->gcache.push_back(gr);
  CK(cudaGraphLaunch(gr.exec, st), "graph launch");
  return VS_OK;
}

// validate, bucket by spot, then K1-K3 over per-spot segments (slices of <= 2^26 items)
vs_status score_device_cells(vs_ctx* c, int64_t n, const int32_t* d_spot, const float* d_q, const float* d_t,
                             float* d_out, cudaStream_t st) {
  const int ns = c->n_spots;
  const int64_t slice = std::max<int64_t>(1, (int64_t(1) << 26) / c->n_lig);
  c->kt_local = 0;
  for (int64_t o = 0; o < n; o += slice) {
    const int64_t nb = std::min(slice, n - o);
    // launch shape from the slice's size (poses spread over the spots: one segment of nb poses approximates it)
    const Shape sh = choose_shape(c, 1, (int)nb);
    const int32_t* sp = d_spot + o;
    const float* q = d_q + 4 * o;
    const float* t = d_t + 3 * o;
    float* out = d_out + o;
    CK(c->buf[B_VALID].ensure(sizeof(int) * nb), "alloc");
    CK(c->buf[B_COUNTS].ensure(sizeof(int) * ns), "alloc");
    CK(c->buf[B_PP].ensure(sizeof(int) * (ns + 1)), "alloc");
    CK(c->buf[B_BP].ensure(sizeof(int) * (ns + 1)), "alloc");
    CK(c->buf[B_CUR].ensure(sizeof(int) * ns), "alloc");
    CK(c->buf[B_SORTED].ensure(sizeof(PoseRec) * nb), "alloc");
    CK(c->buf[B_ORIG].ensure(sizeof(int) * nb), "alloc");
    CK(c->buf[B_PBUF].ensure(sizeof(PoseRec) * nb), "alloc");
    CK(c->buf[B_ITEMS].ensure(sizeof(float4) * nb * c->n_lig), "alloc");
    CK(c->buf[B_E].ensure(sizeof(double) * nb * c->n_lig * sh.nsg()), "alloc");
    int* valid = (int*)c->buf[B_VALID].p;
    int* counts = (int*)c->buf[B_COUNTS].p;
    int* pp = (int*)c->buf[B_PP].p;
    int* cp = (int*)c->buf[B_BP].p;
    int* cur = (int*)c->buf[B_CUR].p;
    PoseRec* sorted = (PoseRec*)c->buf[B_SORTED].p;
    int* orig = (int*)c->buf[B_ORIG].p;
    CK(cudaMemsetAsync(counts, 0, sizeof(int) * ns, st), "memset");
    CK(launch_validate(nb, sp, q, t, ns, c->T, c->all_pairs ? 0 : 1, valid, counts, out, st), "validate launch");
    CK(launch_cell_scan(counts, ns, sh.nn, sh.nh, sh.cn, sh.chb, pp, cp, cur, st), "scan launch");
    CK(launch_scatter(nb, sp, q, t, valid, cur, sorted, orig, st), "scatter launch");
    c->launches += 3;
    CellArgs a = cell_base(c);
    apply_shape(a, sh);
    a.nseg = ns;
    a.seg_spot = c->d_iota;
    a.uniform = 0;
    a.pose_prefix = pp;
    a.chunk_prefix = cp;
    a.mode = MODE_PLAIN;
    a.poses = sorted;
    a.orig = orig;
    a.score_out = out;
    a.pbuf = (PoseRec*)c->buf[B_PBUF].p;
    a.items = (float4*)c->buf[B_ITEMS].p;
    a.E = (double*)c->buf[B_E].p;
    a.E_stride = nb * c->n_lig;
    // pair-kernel grid: an upper bound of sum_k cell_chunks(n_k) (<= n_k n_lig / cn + n_k nh / chb + 3)
    int64_t blocks = 3 * (int64_t)ns + (nb * c->n_lig) / sh.cn + 1;
    if (sh.chb > 0) blocks += (nb * sh.nh) / sh.chb;
    blocks *= sh.nsg();
    if (blocks > 0x7fffffff) return set_err(VS_ERR_INVALID_ARGUMENT, "too many poses in one call");
    vs_status r = cell_launch(c, a, nb, (int)blocks, st);
    if (r != VS_OK) return r;
  }
  if (c->ktime) {
    CK(launch_kt_advance(c->d_kt_base, c->kt_local, st), "kt launch");
    c->launches++;
  }
  return VS_OK;
}

// The asynchronous entry points run on the ctx's own stream, ordered after the caller's stream and before its
// later work by an event pair: the ctx's scratch buffers are then used by one stream only (no overlap between a
// vs_score_poses_device and a vs_run_async of the same ctx), and graph capture always happens on a capturable
// (non-legacy) stream whatever the caller passes (NULL = the legacy default stream included).
vs_status join_in(vs_ctx* c, cudaStream_t caller) {
  CK(cudaEventRecord(c->ev_in, caller), "event record (caller stream)");
  CK(cudaStreamWaitEvent(c->stream, c->ev_in, 0), "stream wait");
  return VS_OK;
}
vs_status join_out(vs_ctx* c, cudaStream_t caller) {
  CK(cudaEventRecord(c->ev_out, c->stream), "event record");
  CK(cudaStreamWaitEvent(caller, c->ev_out, 0), "stream wait (caller stream)");
  return VS_OK;
}

vs_status score_device_impl(vs_ctx* c, int64_t n, const int32_t* d_spot, const float* d_q, const float* d_t,
                            float* d_out, cudaStream_t st) {
  if (n == 0) return VS_OK;
  return score_device_cells(c, n, d_spot, d_q, d_t, d_out, st);
}

}  // namespace

extern "C" {

void vs_score_params_default(vs_score_params* o) {
  if (!o) return;
  o->coulomb_k = 332.0636f;
  o->dielectric = 0;
  o->eps_r = 1.0f;
  o->cutoff = 12.0f;
  o->region_half_width = 3.0f;
  o->hb_eps = 5.0f;
  o->hb_r0 = 1.9f;
  o->r2_min = 0.01f;
  o->n_types = 0;
  o->type_sigma = nullptr;
  o->type_eps = nullptr;
  o->type_hb_role = nullptr;
  o->list_splits = 0;
}

vs_status vs_mh_preset(int m, vs_mh_params* o) {
  if (!o) return set_err(VS_ERR_INVALID_ARGUMENT, "out: NULL");
  if (m < 1 || m > 4) return set_err(VS_ERR_INVALID_ARGUMENT, "preset must be 1..4 (Table 4: M1..M4)");
  o->population = m == 4 ? 1024 : 64;
  o->generations = m == 4 ? 0 : 50;
  o->ls_steps = m == 1 ? 0 : 8;
  o->improve_frac = m == 1 ? 0.0f : (m == 3 ? 0.2f : 1.0f);
  o->p_mut = 0.1f;
  o->mut_trans = 1.0f;
  o->mut_rot = 0.25f;
  o->ls_trans = 0.5f;
  o->ls_rot = 0.10f;
  o->ls_neighbours = 1;
  return VS_OK;
}

vs_status vs_create(const float* rec_xyz, const float* rec_q, const int32_t* rec_type, int32_t n_rec,
                    const float* lig_xyz, const float* lig_q, const int32_t* lig_type, int32_t n_lig,
                    const float* spot_xyz, int32_t n_spots, const vs_score_params* sp_in, int32_t cuda_device,
                    vs_ctx** out) {
  if (!out) return set_err(VS_ERR_INVALID_ARGUMENT, "out: NULL");
  *out = nullptr;
  if (!rec_xyz || !rec_q || !rec_type || !lig_xyz || !lig_q || !lig_type || !spot_xyz)
    return set_err(VS_ERR_INVALID_ARGUMENT, "NULL input array");
  if (n_rec < 1 || n_lig < 1 || n_lig > 256 || n_spots < 1)
    return set_err(VS_ERR_INVALID_ARGUMENT, "need n_rec >= 1, 1 <= n_lig <= 256, n_spots >= 1");
  vs_score_params sp;
  if (sp_in) sp = *sp_in; else vs_score_params_default(&sp);
  if (!std::isfinite(sp.coulomb_k) || (sp.dielectric != 0 && sp.dielectric != 1) ||
      (sp.dielectric == 1 && !(sp.eps_r > 0.0f && std::isfinite(sp.eps_r))) ||
      !(sp.region_half_width > 0.0f && std::isfinite(sp.region_half_width)) ||
      !(sp.hb_eps >= 0.0f && std::isfinite(sp.hb_eps)) || !(sp.hb_r0 > 0.0f && std::isfinite(sp.hb_r0)) ||
      !(sp.r2_min > 0.0f && std::isfinite(sp.r2_min)) || std::isnan(sp.cutoff))
    return set_err(VS_ERR_INVALID_ARGUMENT, "invalid score params");
  // list_splits 0 = by the context's spot count: few spots -> latency-bound runs -> more splits (R32)
  if (sp.list_splits == 0) sp.list_splits = n_spots <= 96 ? 4 : (n_spots <= 200 ? 2 : 1);
  if (sp.list_splits != 1 && sp.list_splits != 2 && sp.list_splits != 4)
    return set_err(VS_ERR_INVALID_ARGUMENT, "list_splits must be 0, 1, 2 or 4");
  if (sp.n_types < 0 || sp.n_types > 64 || (sp.n_types > 0 && (!sp.type_sigma || !sp.type_eps || !sp.type_hb_role)))
    return set_err(VS_ERR_INVALID_ARGUMENT, "invalid type table");
  if (!finite_arr(rec_xyz, 3 * (int64_t)n_rec) || !finite_arr(rec_q, n_rec) || !finite_arr(lig_xyz, 3 * (int64_t)n_lig) ||
      !finite_arr(lig_q, n_lig) || !finite_arr(spot_xyz, 3 * (int64_t)n_spots))
    return set_err(VS_ERR_INVALID_ARGUMENT, "non-finite input");
  const int nt = sp.n_types > 0 ? sp.n_types : 7;
  std::vector<float> c12(nt), c6(nt), don(nt), acc(nt);
  for (int t = 0; t < nt; ++t) {
    const float sg = sp.n_types > 0 ? sp.type_sigma[t] : kSigma[t];
    const float ep = sp.n_types > 0 ? sp.type_eps[t] : kEps[t];
    const int rl = sp.n_types > 0 ? sp.type_hb_role[t] : kRole[t];
    if (!(sg >= 0.0f && std::isfinite(sg)) || !(ep >= 0.0f && std::isfinite(ep)) || rl < 0 || rl > 2)
      return set_err(VS_ERR_INVALID_ARGUMENT, "invalid type table entry");
    // geometric combining: 4 eps_ij (sig_ij^12/r^12 - sig_ij^6/r^6) = c12_i c12_j/r^12 - c6_i c6_j/r^6 (R4)
    c12[t] = (float)(2.0 * std::sqrt((double)ep) * std::pow((double)sg, 6));
    c6[t] = (float)(2.0 * std::sqrt((double)ep) * std::pow((double)sg, 3));
    don[t] = rl == 1 ? 1.0f : 0.0f;
    acc[t] = rl == 2 ? 1.0f : 0.0f;
  }
  for (int i = 0; i < n_rec; ++i)
    if (rec_type[i] < 0 || rec_type[i] >= nt) return set_err(VS_ERR_INVALID_ARGUMENT, "receptor type id out of range");
  for (int i = 0; i < n_lig; ++i)
    if (lig_type[i] < 0 || lig_type[i] >= nt) return set_err(VS_ERR_INVALID_ARGUMENT, "ligand type id out of range");

  int ndev = 0;
  cudaError_t e0 = cudaGetDeviceCount(&ndev);
  if (e0 != cudaSuccess || ndev == 0)
    return set_err(VS_ERR_CUDA, std::string("no CUDA device: ") + cudaGetErrorString(e0));
  if (cuda_device < 0 || cuda_device >= ndev) return set_err(VS_ERR_INVALID_ARGUMENT, "cuda_device out of range");

  vs_ctx* c = new (std::nothrow) vs_ctx;
  if (!c) return set_err(VS_ERR_OUT_OF_MEMORY, "out of host memory");
  DeviceGuard guard(cuda_device);
  c->dev = cuda_device;
  {
    int nsm = 0;
    if (cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, cuda_device) == cudaSuccess && nsm > 0)
      c->n_sm = nsm;
  }
  c->n_rec = n_rec;
  c->n_lig = n_lig;
  c->n_spots = n_spots;
  // launch-shape knobs for experiments (speed only; results never depend on them)
  if (const char* v = std::getenv("VS_FILL_WARPS")) c->fill_warps = std::max(1ll, std::atoll(v));
  if (const char* v = std::getenv("VS_DIRECT_GROUP_SPOTS")) c->direct_group_spots = std::max(1, std::atoi(v));
  if (const char* v = std::getenv("VS_TRIGGER_SPOTS")) c->trigger_spots = std::atoi(v);
  if (const char* v = std::getenv("VS_SHAPE")) {  // "kp"
    const int kp = std::atoi(v);
    if (kp == 1 || kp == 2) c->force_kp = kp;
  }
  c->all_pairs = !(sp.cutoff > 0.0f) || std::isinf(sp.cutoff);
  c->dielectric = sp.dielectric;
  c->nsplit = sp.list_splits;
  c->T = sp.region_half_width;
  c->rc = c->all_pairs ? INFINITY : sp.cutoff;
  c->rc2 = c->all_pairs ? INFINITY : (float)((double)sp.cutoff * sp.cutoff);
  c->inv_rc2 = c->all_pairs ? 0.0f : (float)(1.0 / ((double)sp.cutoff * sp.cutoff));
  c->r2min = sp.r2_min;
  c->hbC = (float)(5.0 * sp.hb_eps * std::pow((double)sp.hb_r0, 12));
  c->hbD = (float)(6.0 * sp.hb_eps * std::pow((double)sp.hb_r0, 10));

  auto fail = [&](vs_status s) {
    vs_destroy(c);
    return s;
  };
#define CKC(expr, where)                                     \
  do {                                                       \
    cudaError_t e_ = (expr);                                 \
    if (e_ != cudaSuccess) return fail(cuda_fail(nullptr, e_, where)); \
  } while (0)

  CKC(cudaStreamCreateWithFlags(&c->stream, cudaStreamNonBlocking), "stream create");
  for (int i = 0; i < NSUB; ++i) {
    CKC(cudaStreamCreateWithFlags(&c->sub[i], cudaStreamNonBlocking), "stream create");
    CKC(cudaEventCreateWithFlags(&c->ev_join[i], cudaEventDisableTiming), "event create");
  }
  CKC(cudaEventCreateWithFlags(&c->ev_fork, cudaEventDisableTiming), "event create");
  CKC(cudaEventCreateWithFlags(&c->ev_in, cudaEventDisableTiming), "event create");
  CKC(cudaEventCreateWithFlags(&c->ev_out, cudaEventDisableTiming), "event create");
  // ligand: centred on the fp32-rounded fp64 centroid (R11)
  float cen[3];
  for (int a = 0; a < 3; ++a) {
    double s = 0.0;
    for (int i = 0; i < n_lig; ++i) s += lig_xyz[3 * i + a];
    cen[a] = (float)(s / n_lig);
  }
  // radius of the centred ligand (list reach, R10; item sort grid)
  double rmax = 0.0;
  for (int i = 0; i < n_lig; ++i) {
    const double x = (float)(lig_xyz[3 * i] - cen[0]), y = (float)(lig_xyz[3 * i + 1] - cen[1]),
                 z = (float)(lig_xyz[3 * i + 2] - cen[2]);
    rmax = std::max(rmax, std::sqrt(x * x + y * y + z * z));
  }
  {
    // ligand atoms in input order; class 1 = H-bond role (donor / acceptor, R5)
    std::vector<float4> lx(n_lig), lp(n_lig);
    std::vector<int> rank(n_lig);
    int cnt[2] = {0, 0};
    bool any_role = false;  // a ligand without H-bond atoms keeps H = 0 (no H-bond slots) even with VS_CELL_MERGE
    for (int i = 0; i < n_lig; ++i) any_role = any_role || don[lig_type[i]] != 0.0f || acc[lig_type[i]] != 0.0f;
    // one item class for every launch ("merge": every atom in the H-bond slots, one curve order, spatially tighter
    // slot pairs at 23 instead of 19 issue slots for class-0 pairs): measured large -2.5 %, medium +2.3 %, sweep
    // +2.5 % (profiles/r02_notes.md), so off by default; KP = 1 launches merge anyway (shape_of).  Layout only: the
    // item order never enters a result.  VS_CELL_MERGE=0/1 (environment) forces it.
    int merge_mode = VS_CELL_MERGE;
    if (const char* v = std::getenv("VS_CELL_MERGE")) merge_mode = std::atoi(v);
    const bool merge = merge_mode && any_role;
    for (int i = 0; i < n_lig; ++i) {
      const int t = lig_type[i];
      const int role = (don[t] != 0.0f || acc[t] != 0.0f) ? 1 : 0;
      // item class (K1 sorts and chunks the classes apart; class-1 items sit in H-bond slots): the H-bond role, or
      // class 1 for every atom with VS_CELL_MERGE (one curve order for all items, all slots H-bond slots).  ligx.w
      // = 0 class 0; 1 class 1 with an H-bond role; 2 class 1 without one (its H-bond sums are discarded)
      const int cls = merge ? 1 : role;
      lx[i] = make_float4(lig_xyz[3 * i] - cen[0], lig_xyz[3 * i + 1] - cen[1], lig_xyz[3 * i + 2] - cen[2],
                          cls == 0 ? 0.0f : (role ? 1.0f : 2.0f));
      const double qk = sp.dielectric == 0 ? (double)sp.coulomb_k * lig_q[i] / 4.0
                                           : (double)sp.coulomb_k * lig_q[i] / (double)sp.eps_r;
      lp[i] = make_float4((float)qk, c12[t], c6[t], don[t]);
      rank[i] = cnt[cls]++;
    }
    c->nn = cnt[0];
    c->nh = cnt[1];
    // H-bond slot pairs per lane of the KP = 2 kernel: the H minimising (chunks per pose) x (issue slots per
    // chunk), with 19 slots per class-0-only pair and 23 per H-bond pair; class-0 items may
    // overflow into H-bond slots, so chunks per pose = max(n / CH_ITEMS, nh / (64 H)).  The KP = 1 kernel has
    // one slot pair: an H-bond pair whenever the ligand has H-bond atoms.
    double best = 1e300;
    for (int h = merge ? CELL_KP : 0; h <= CELL_KP; ++h) {
      if (c->nh > 0 && h == 0) continue;
      const double per = std::max((double)n_lig / CH_ITEMS, h > 0 ? c->nh / (64.0 * h) : 0.0);
      const double cost = per * (19.0 * (CELL_KP - h) + 23.0 * h);
      if (cost < best - 1e-12) {
        best = cost;
        c->H2 = h;
      }
    }
    c->H1 = c->nh > 0 ? 1 : 0;
    CKC(pool::alloc(&c->d_ligx, sizeof(float4) * n_lig), "alloc ligand");
    CKC(pool::alloc(&c->d_ligp, sizeof(float4) * n_lig), "alloc ligand");
    CKC(pool::alloc(&c->d_lig_rank, sizeof(int) * n_lig), "alloc ligand");
    CKC(cudaMemcpyAsync(c->d_ligx, lx.data(), sizeof(float4) * n_lig, cudaMemcpyHostToDevice, c->stream), "H2D ligand");
    CKC(cudaMemcpyAsync(c->d_ligp, lp.data(), sizeof(float4) * n_lig, cudaMemcpyHostToDevice, c->stream), "H2D ligand");
    CKC(cudaMemcpyAsync(c->d_lig_rank, rank.data(), sizeof(int) * n_lig, cudaMemcpyHostToDevice, c->stream), "H2D ligand");
  }

  // receptor atoms (absolute) + per-atom parameters
  std::vector<float4> hrec(n_rec), hprm(n_rec);
  for (int j = 0; j < n_rec; ++j) {
    const int t = rec_type[j];
    hrec[j] = make_float4(rec_xyz[3 * j], rec_xyz[3 * j + 1], rec_xyz[3 * j + 2], rec_q[j]);
    hprm[j] = make_float4(c12[t], c6[t], don[t], acc[t]);
  }
  float4* d_rec = nullptr;
  float4* d_prm = nullptr;
  float4* d_centres = nullptr;
  auto free_tmp = [&]() {
    cudaStreamSynchronize(c->stream);  // list-building launches may still read the temporaries
    if (d_rec) pool::release(d_rec);
    if (d_prm) pool::release(d_prm);
    if (d_centres) pool::release(d_centres);
  };
#define CKT(expr, where)                                                       \
  do {                                                                         \
    cudaError_t e_ = (expr);                                                   \
    if (e_ != cudaSuccess) { free_tmp(); return fail(cuda_fail(nullptr, e_, where)); } \
  } while (0)
  CKT(pool::alloc(&d_rec, sizeof(float4) * n_rec), "alloc receptor");
  CKT(pool::alloc(&d_prm, sizeof(float4) * n_rec), "alloc receptor");
  CKT(cudaMemcpyAsync(d_rec, hrec.data(), sizeof(float4) * n_rec, cudaMemcpyHostToDevice, c->stream), "H2D receptor");
  CKT(cudaMemcpyAsync(d_prm, hprm.data(), sizeof(float4) * n_rec, cudaMemcpyHostToDevice, c->stream), "H2D receptor");

  std::vector<int> h_off(n_spots), h_len(n_spots), iota(n_spots);
  std::vector<float4> h_shift(n_spots);
  for (int s = 0; s < n_spots; ++s) iota[s] = s;
  if (c->all_pairs) {
    // every spot streams the whole receptor, stored relative to the spot centre (fp32 r_j - c_s,
    // the same relative frame as the cutoff lists: keeps the pair differences accurate)
    std::vector<float4> hc(n_spots);
    for (int s = 0; s < n_spots; ++s) hc[s] = make_float4(spot_xyz[3 * s], spot_xyz[3 * s + 1], spot_xyz[3 * s + 2], 0.0f);
    CKT(pool::alloc(&d_centres, sizeof(float4) * n_spots), "alloc");
    CKT(cudaMemcpyAsync(d_centres, hc.data(), sizeof(float4) * n_spots, cudaMemcpyHostToDevice, c->stream), "H2D");
    const int64_t tot = (int64_t)n_rec * n_spots;
    if (tot > 0x7fffffff) { free_tmp(); return fail(set_err(VS_ERR_OUT_OF_MEMORY, "receptor lists exceed 2^31 atoms")); }
    for (int s = 0; s < n_spots; ++s) {
      h_off[s] = (int)((int64_t)s * n_rec);
      h_len[s] = n_rec;
      h_shift[s] = make_float4(0, 0, 0, 0);
    }
    CKT(pool::alloc(&c->d_lists, sizeof(RecAtom) * tot), "alloc lists");
    CKT(pool::alloc(&c->d_list_off, sizeof(int) * n_spots), "alloc");
    CKT(cudaMemcpyAsync(c->d_list_off, h_off.data(), sizeof(int) * n_spots, cudaMemcpyHostToDevice, c->stream), "H2D");
    CKT(launch_build_lists(d_rec, d_prm, n_rec, d_centres, n_spots, INFINITY, c->d_list_off, nullptr, c->d_lists, 0,
                           c->stream), "list fill launch");
    c->list_total = tot;
  } else {
    // per-spot lists: atoms within T sqrt(3) + max|l_i| + rc + 0.01 of the spot centre (R10)
    const double reach = (double)c->T * std::sqrt(3.0) + rmax + (double)sp.cutoff + 0.01;
    std::vector<float4> hc(n_spots);
    for (int s = 0; s < n_spots; ++s) hc[s] = make_float4(spot_xyz[3 * s], spot_xyz[3 * s + 1], spot_xyz[3 * s + 2], 0.0f);
    CKT(pool::alloc(&d_centres, sizeof(float4) * n_spots), "alloc");
    CKT(cudaMemcpyAsync(d_centres, hc.data(), sizeof(float4) * n_spots, cudaMemcpyHostToDevice, c->stream), "H2D");
    CKT(pool::alloc(&c->d_list_len, sizeof(int) * n_spots), "alloc");
    CKT(pool::alloc(&c->d_list_off, sizeof(int) * n_spots), "alloc");
    CKT(launch_build_lists(d_rec, d_prm, n_rec, d_centres, n_spots, (float)(reach * reach), nullptr, c->d_list_len,
                           nullptr, 1, c->stream), "list count launch");
    CKT(cudaMemcpyAsync(h_len.data(), c->d_list_len, sizeof(int) * n_spots, cudaMemcpyDeviceToHost, c->stream), "D2H");
    CKT(cudaStreamSynchronize(c->stream), "sync");
    int64_t tot = 0;
    for (int s = 0; s < n_spots; ++s) {
      h_off[s] = (int)tot;
      tot += h_len[s];
      h_shift[s] = make_float4(0, 0, 0, 0);
    }
    if (tot > 0x7fffffff) { free_tmp(); return fail(set_err(VS_ERR_OUT_OF_MEMORY, "receptor lists exceed 2^31 atoms")); }
    c->list_total = tot;
    CKT(pool::alloc(&c->d_lists, sizeof(RecAtom) * std::max<int64_t>(tot, 1)), "alloc lists");
    CKT(cudaMemcpyAsync(c->d_list_off, h_off.data(), sizeof(int) * n_spots, cudaMemcpyHostToDevice, c->stream), "H2D");
    CKT(launch_build_lists(d_rec, d_prm, n_rec, d_centres, n_spots, (float)(reach * reach), c->d_list_off, nullptr,
                           c->d_lists, 0, c->stream), "list fill launch");
    // cell-sorted lists + cell start table (per-chunk culling in the pair kernel)
    CKT(cudaMemcpyAsync(c->d_list_len, h_len.data(), sizeof(int) * n_spots, cudaMemcpyHostToDevice, c->stream), "H2D");
    RecAtom* sorted = nullptr;
    CKT(pool::alloc(&sorted, sizeof(RecAtom) * std::max<int64_t>(tot, 1)), "alloc lists");
    c->cR = (float)reach + 0.01f;
    c->cell_g = cell_grid(c->nsplit);
    if (const char* v = std::getenv("VS_CELL_GRID")) {  // tests / experiments: force the grid (speed only)
      const int g = std::atoi(v);
      if (g >= 4 && g <= CELL_GMAX && g % c->nsplit == 0) c->cell_g = g;
    }
    const int G = c->cell_g;
    c->ch = 2.0f * c->cR / (float)G;
    c->cinv_h = (float)G / (2.0f * c->cR);
    CKT(pool::alloc(&c->d_cells, sizeof(uint16_t) * (size_t)n_spots * ((size_t)G * G * G + 1)), "alloc cell tables");
    cudaError_t es = launch_cell_sort(c->d_lists, sorted, c->d_list_off, c->d_list_len, n_spots, c->d_cells, G,
                                      c->cR, c->cinv_h, c->stream);
    if (es == cudaSuccess) es = cudaStreamSynchronize(c->stream);
    pool::release(c->d_lists);
    c->d_lists = sorted;
    CKT(es, "list sort launch");
  }
  if (!c->d_list_len) CKT(pool::alloc(&c->d_list_len, sizeof(int) * n_spots), "alloc");
  CKT(cudaMemcpyAsync(c->d_list_len, h_len.data(), sizeof(int) * n_spots, cudaMemcpyHostToDevice, c->stream), "H2D");
  CKT(cudaMemcpyAsync(c->d_list_off, h_off.data(), sizeof(int) * n_spots, cudaMemcpyHostToDevice, c->stream), "H2D");
  c->W = c->T + (float)rmax + 0.01f;  // cutoff mode: |x_k| <= T + max|l_i| for every transformed atom
  c->inv_hm = (float)(1 << MORTON_BITS) / (2.0f * c->W);
  CKT(pool::alloc(&c->d_shift, sizeof(float4) * n_spots), "alloc");
  CKT(cudaMemcpyAsync(c->d_shift, h_shift.data(), sizeof(float4) * n_spots, cudaMemcpyHostToDevice, c->stream), "H2D");
  CKT(pool::alloc(&c->d_iota, sizeof(int) * n_spots), "alloc");
  CKT(cudaMemcpyAsync(c->d_iota, iota.data(), sizeof(int) * n_spots, cudaMemcpyHostToDevice, c->stream), "H2D");
  CKT(pool::alloc(&c->d_counters, sizeof(unsigned long long) * 4), "alloc");
  CKT(pool::alloc(&c->d_seed, sizeof(uint64_t)), "alloc");
  {
    const char* gv = std::getenv("VS_GRAPHS");
    c->graphs = !(gv && gv[0] == '0');
  }
  CKT(cudaMemset(c->d_counters, 0, sizeof(unsigned long long) * 4), "memset");
  CKT(cudaStreamSynchronize(c->stream), "sync");
  free_tmp();
  c->h_list_len = h_len;
  c->launches = 0;
  *out = c;
  return VS_OK;
#undef CKT
#undef CKC
}

vs_status vs_score_poses(vs_ctx* c, int64_t n, const int32_t* spot, const float* q, const float* t, float* out) {
  if (!c) return set_err(VS_ERR_INVALID_ARGUMENT, "ctx: NULL");
  if (c->poisoned) return set_err(VS_ERR_CUDA, "ctx poisoned by an earlier CUDA error");
  if (n < 0) return set_err(VS_ERR_INVALID_ARGUMENT, "n must be >= 0");
  if (n == 0) return VS_OK;
  if (!spot || !q || !t || !out) return set_err(VS_ERR_INVALID_ARGUMENT, "NULL pose array");
  for (int64_t p = 0; p < n; ++p) {
    if (spot[p] < 0 || spot[p] >= c->n_spots) return set_err(VS_ERR_INVALID_ARGUMENT, "spot id out of range");
    if (!finite_arr(q + 4 * p, 4) || !finite_arr(t + 3 * p, 3)) return set_err(VS_ERR_INVALID_ARGUMENT, "non-finite pose");
    if (q[4 * p] == 0.0f && q[4 * p + 1] == 0.0f && q[4 * p + 2] == 0.0f && q[4 * p + 3] == 0.0f)
      return set_err(VS_ERR_ZERO_QUATERNION, "zero quaternion");
    if (!c->all_pairs)
      for (int a = 0; a < 3; ++a)
        if (std::fabs(t[3 * p + a]) > c->T) return set_err(VS_ERR_POSE_OUT_OF_REGION, "translation outside the spot region");
  }
  DeviceGuard guard(c->dev);
  cudaStream_t st = c->stream;
  CK(c->buf[B_SPOT].ensure(sizeof(int32_t) * n), "alloc");
  CK(c->buf[B_Q].ensure(sizeof(float) * 4 * n), "alloc");
  CK(c->buf[B_T].ensure(sizeof(float) * 3 * n), "alloc");
  CK(c->buf[B_OUT].ensure(sizeof(float) * n), "alloc");
  CK(cudaMemcpyAsync(c->buf[B_SPOT].p, spot, sizeof(int32_t) * n, cudaMemcpyHostToDevice, st), "H2D");
  CK(cudaMemcpyAsync(c->buf[B_Q].p, q, sizeof(float) * 4 * n, cudaMemcpyHostToDevice, st), "H2D");
  CK(cudaMemcpyAsync(c->buf[B_T].p, t, sizeof(float) * 3 * n, cudaMemcpyHostToDevice, st), "H2D");
  vs_status s = score_device_impl(c, n, (const int32_t*)c->buf[B_SPOT].p, (const float*)c->buf[B_Q].p,
                                  (const float*)c->buf[B_T].p, (float*)c->buf[B_OUT].p, st);
  if (s != VS_OK) return s;
  CK(cudaMemcpyAsync(out, c->buf[B_OUT].p, sizeof(float) * n, cudaMemcpyDeviceToHost, st), "D2H");
  CK(cudaStreamSynchronize(st), "sync");
  return VS_OK;
}

vs_status vs_score_poses_device(vs_ctx* c, int64_t n, const int32_t* d_spot, const float* d_q, const float* d_t,
                                float* d_score, void* stream) {
  if (!c) return set_err(VS_ERR_INVALID_ARGUMENT, "ctx: NULL");
  if (c->poisoned) return set_err(VS_ERR_CUDA, "ctx poisoned by an earlier CUDA error");
  if (n < 0) return set_err(VS_ERR_INVALID_ARGUMENT, "n must be >= 0");
  if (n == 0) return VS_OK;
  if (!d_spot || !d_q || !d_t || !d_score) return set_err(VS_ERR_INVALID_ARGUMENT, "NULL pose array");
  DeviceGuard guard(c->dev);
  vs_status r = join_in(c, (cudaStream_t)stream);
  if (r == VS_OK) r = score_device_impl(c, n, d_spot, d_q, d_t, d_score, c->stream);
  if (r == VS_OK) r = join_out(c, (cudaStream_t)stream);
  return r;
}

static vs_status run_host(vs_ctx* c, const vs_mh_params* mp, uint64_t seed, int32_t n_sel, const int32_t* spot_ids,
                          float* best_pose, float* best_score, Tracer* tr) {
  if (!c) return set_err(VS_ERR_INVALID_ARGUMENT, "ctx: NULL");
  if (c->poisoned) return set_err(VS_ERR_CUDA, "ctx poisoned by an earlier CUDA error");
  if (!best_pose || !best_score) return set_err(VS_ERR_INVALID_ARGUMENT, "NULL output");
  DeviceGuard guard(c->dev);
  const int ns = spot_ids ? n_sel : c->n_spots;
  if (ns < 0) return set_err(VS_ERR_INVALID_ARGUMENT, "n_sel must be >= 0");
  CK(c->buf[B_BEST].ensure(sizeof(float) * 7 * std::max(ns, 1)), "alloc");
  CK(c->buf[B_BESTS].ensure(sizeof(float) * std::max(ns, 1)), "alloc");
  vs_status s = run_impl(c, mp, seed, n_sel, spot_ids, (float*)c->buf[B_BEST].p, (float*)c->buf[B_BESTS].p,
                         c->stream, tr);
  if (s != VS_OK) return s;
  CK(cudaMemcpyAsync(best_pose, c->buf[B_BEST].p, sizeof(float) * 7 * ns, cudaMemcpyDeviceToHost, c->stream), "D2H");
  CK(cudaMemcpyAsync(best_score, c->buf[B_BESTS].p, sizeof(float) * ns, cudaMemcpyDeviceToHost, c->stream), "D2H");
  CK(cudaStreamSynchronize(c->stream), "sync");
  return VS_OK;
}

vs_status vs_run(vs_ctx* c, const vs_mh_params* mp, uint64_t seed, int32_t n_sel, const int32_t* spot_ids,
                 float* best_pose_out, float* best_score_out) {
  return run_host(c, mp, seed, n_sel, spot_ids, best_pose_out, best_score_out, nullptr);
}

vs_status vs_run_trace(vs_ctx* c, const vs_mh_params* mp, uint64_t seed, int32_t n_sel, const int32_t* spot_ids,
                       float* best_pose_out, float* best_score_out, vs_trace_fn fn, void* user) {
  Tracer tr;
  tr.fn = fn;
  tr.user = user;
  return run_host(c, mp, seed, n_sel, spot_ids, best_pose_out, best_score_out, &tr);
}

vs_status vs_run_async(vs_ctx* c, const vs_mh_params* mp, uint64_t seed, int32_t n_sel, const int32_t* spot_ids,
                       float* d_best_pose, float* d_best_score, void* stream) {
  if (!c) return set_err(VS_ERR_INVALID_ARGUMENT, "ctx: NULL");
  if (c->poisoned) return set_err(VS_ERR_CUDA, "ctx poisoned by an earlier CUDA error");
  if (!d_best_pose || !d_best_score) return set_err(VS_ERR_INVALID_ARGUMENT, "NULL output");
  DeviceGuard guard(c->dev);
  vs_status r = join_in(c, (cudaStream_t)stream);
  if (r == VS_OK) r = run_impl(c, mp, seed, n_sel, spot_ids, d_best_pose, d_best_score, c->stream, nullptr);
  if (r == VS_OK) r = join_out(c, (cudaStream_t)stream);
  return r;
}

// VS_DEBUG_TIMING=1: phase times of vs_destroy on stderr (host-side cost investigation)
static bool debug_timing() {
  static const bool on = std::getenv("VS_DEBUG_TIMING") != nullptr;
  return on;
}

void vs_destroy(vs_ctx* c) {
  if (!c) return;
  DeviceGuard guard(c->dev);
  using clk = std::chrono::steady_clock;
  auto t = clk::now();
  double ph[6] = {0, 0, 0, 0, 0, 0};
  auto lap = [&](int i) {
    const auto n = clk::now();
    ph[i] = std::chrono::duration<double, std::milli>(n - t).count();
    t = n;
  };
  if (c->stream) cudaStreamSynchronize(c->stream);
  cudaDeviceSynchronize();
  lap(0);
  for (auto& b : c->buf) b.release();
  lap(1);
  for (auto e : c->ev) cudaEventDestroy(e);
  for (auto& gr : c->gcache) cudaGraphExecDestroy(gr.exec);
  lap(2);
  void* ptrs[] = {c->d_lists, c->d_list_off, c->d_list_len, c->d_shift, c->d_iota, c->d_counters,
                  c->d_seed, c->d_cells, c->d_ligx, c->d_ligp, c->d_lig_rank, c->d_kt, c->d_kt_base};
  for (void* p : ptrs)
    if (p) pool::release(p);
  lap(3);
  if (c->stream) cudaStreamDestroy(c->stream);
  for (int i = 0; i < NSUB; ++i) {
    if (c->sub[i]) cudaStreamDestroy(c->sub[i]);
    if (c->ev_join[i]) cudaEventDestroy(c->ev_join[i]);
  }
  if (c->ev_fork) cudaEventDestroy(c->ev_fork);
  if (c->ev_in) cudaEventDestroy(c->ev_in);
  if (c->ev_out) cudaEventDestroy(c->ev_out);
  lap(4);
  delete c;
  if (debug_timing())
    std::fprintf(stderr, "vs_destroy ms: sync %.2f bufs %.2f events+graph %.2f frees %.2f streams %.2f\n", ph[0], ph[1],
                 ph[2], ph[3], ph[4]);
}

vs_status vs_release_cached_memory(int32_t cuda_device) {
  int n = 0;
  if (cudaGetDeviceCount(&n) != cudaSuccess) n = 0;
  if (cuda_device >= n) return set_err(VS_ERR_INVALID_ARGUMENT, "no such CUDA device");
  std::vector<int> devs;
  {
    std::lock_guard<std::mutex> g(pool::mu);
    for (auto& kv : pool::devs())
      if (cuda_device < 0 || kv.first == cuda_device) devs.push_back(kv.first);
  }
  for (int d : devs) {
    DeviceGuard guard(d);
    pool::trim(d);
  }
  return VS_OK;
}

const char* vs_last_error(void) { return g_err.c_str(); }
int vs_abi_version(void) { return VS_ABI_VERSION; }

vs_status vs_set_timing(vs_ctx* c, int flags) {
  if (!c) return set_err(VS_ERR_INVALID_ARGUMENT, "ctx: NULL");
  if (c->poisoned) return set_err(VS_ERR_CUDA, "ctx poisoned by an earlier CUDA error");
  DeviceGuard guard(c->dev);
  if ((flags & VS_TIMING_KERNEL) && !c->d_kt) {
    CK(cudaStreamSynchronize(c->stream), "sync");
    CK(pool::alloc(&c->d_kt, sizeof(unsigned long long) * KT_WORDS * (size_t)VS_KT_CAP), "alloc");
    CK(pool::alloc(&c->d_kt_base, sizeof(unsigned long long)), "alloc");
    CK(cudaMemset(c->d_kt, 0, sizeof(unsigned long long) * KT_WORDS * (size_t)VS_KT_CAP), "memset");
    CK(cudaMemset(c->d_kt_base, 0, sizeof(unsigned long long)), "memset");
  }
  c->timing = (flags & VS_TIMING_EVENTS) != 0;
  c->ktime = (flags & VS_TIMING_KERNEL) != 0;
  c->census = (flags & VS_TIMING_CENSUS) != 0;
  return VS_OK;
}

vs_status vs_get_stats(vs_ctx* c, vs_stats* o) {
  if (!c || !o) return set_err(VS_ERR_INVALID_ARGUMENT, "NULL argument");
  if (c->poisoned) return set_err(VS_ERR_CUDA, "ctx poisoned by an earlier CUDA error");
  DeviceGuard guard(c->dev);
  CK(cudaDeviceSynchronize(), "sync");
  vs_status s = collect_timing(c);
  if (s != VS_OK) return s;
  unsigned long long h[4];
  CK(cudaMemcpy(h, c->d_counters, sizeof(h), cudaMemcpyDeviceToHost), "D2H counters");
  h[1] += c->host_poses;
  h[2] += c->host_pairs;
  o->pairs_within = c->all_pairs ? h[2] : h[3];  // all-pairs mode: every pair is within
  o->pair_busy_ms = o->pair_launch_ms = o->pair_warp_ms = 0.0;
  o->pair_timed_launches = 0;
  if (c->d_kt) {  // pair-kernel launch intervals: their sum and the length of their union
    unsigned long long nslot = 0;
    CK(cudaMemcpy(&nslot, c->d_kt_base, sizeof(nslot), cudaMemcpyDeviceToHost), "D2H kt");
    nslot = std::min<unsigned long long>(nslot, VS_KT_CAP);
    std::vector<unsigned long long> kt(KT_WORDS * nslot);
    if (nslot)
      CK(cudaMemcpy(kt.data(), c->d_kt, sizeof(unsigned long long) * KT_WORDS * nslot, cudaMemcpyDeviceToHost), "D2H kt");
    std::vector<std::pair<unsigned long long, unsigned long long>> iv;
    double warp_ns = 0.0;
    for (unsigned long long i = 0; i < nslot; ++i)
      if (kt[KT_WORDS * i] && kt[KT_WORDS * i + 1]) {
        iv.emplace_back(~kt[KT_WORDS * i], kt[KT_WORDS * i + 1]);
        warp_ns += (double)kt[KT_WORDS * i + 2];
      }
    o->pair_warp_ms = warp_ns * 1e-6;
    std::sort(iv.begin(), iv.end());
    double sum = 0.0, busy = 0.0;
    unsigned long long cs = 0, ce = 0;
    bool open = false;
    for (auto& x : iv) {
      if (x.second < x.first) continue;
      sum += (double)(x.second - x.first);
      if (!open || x.first > ce) {
        if (open) busy += (double)(ce - cs);
        cs = x.first;
        ce = x.second;
        open = true;
      } else if (x.second > ce) {
        ce = x.second;
      }
    }
    if (open) busy += (double)(ce - cs);
    o->pair_busy_ms = busy * 1e-6;
    o->pair_launch_ms = sum * 1e-6;
    o->pair_timed_launches = iv.size();
  }
  o->kernel_launches = c->launches;
  o->score_launches = c->score_launches;
  o->pairs = h[2];
  o->poses_scored = h[1];
  o->pairs_evaluated = h[0];
  o->score_ms = c->score_ms_acc;
  o->timed_launches = c->timed_acc;
  return VS_OK;
}

vs_status vs_reset_stats(vs_ctx* c) {
  if (!c) return set_err(VS_ERR_INVALID_ARGUMENT, "ctx: NULL");
  if (c->poisoned) return set_err(VS_ERR_CUDA, "ctx poisoned by an earlier CUDA error");
  DeviceGuard guard(c->dev);
  CK(cudaDeviceSynchronize(), "sync");
  CK(cudaMemset(c->d_counters, 0, sizeof(unsigned long long) * 4), "memset");
  c->host_poses = c->host_pairs = 0;
  if (c->d_kt) {
    CK(cudaMemset(c->d_kt, 0, sizeof(unsigned long long) * KT_WORDS * (size_t)VS_KT_CAP), "memset");
    CK(cudaMemset(c->d_kt_base, 0, sizeof(unsigned long long)), "memset");
  }
  c->ev_used = 0;
  c->launches = c->score_launches = 0;
  c->score_ms_acc = 0.0;
  c->timed_acc = 0;
  return VS_OK;
}

int64_t vs_pair_intervals(vs_ctx* c, uint64_t* out, int64_t cap) {
  if (!c || cap < 0 || (cap > 0 && !out)) {
    set_err(VS_ERR_INVALID_ARGUMENT, "bad arguments");
    return -1;
  }
  if (c->poisoned || !c->d_kt) return 0;
  DeviceGuard guard(c->dev);
  if (cudaDeviceSynchronize() != cudaSuccess) return -1;
  unsigned long long nslot = 0;
  if (cudaMemcpy(&nslot, c->d_kt_base, sizeof(nslot), cudaMemcpyDeviceToHost) != cudaSuccess) return -1;
  nslot = std::min<unsigned long long>(nslot, VS_KT_CAP);
  std::vector<unsigned long long> kt(KT_WORDS * nslot);
  if (nslot && cudaMemcpy(kt.data(), c->d_kt, sizeof(unsigned long long) * KT_WORDS * nslot, cudaMemcpyDeviceToHost) !=
                   cudaSuccess)
    return -1;
  int64_t n = 0;
  for (unsigned long long i = 0; i < nslot; ++i)
    if (kt[KT_WORDS * i] && kt[KT_WORDS * i + 1] && kt[KT_WORDS * i + 1] >= ~kt[KT_WORDS * i]) {
      if (n < cap) {
        out[2 * n] = ~kt[KT_WORDS * i];
        out[2 * n + 1] = kt[KT_WORDS * i + 1];
      }
      ++n;
    }
  return n;
}

vs_status vs_list_lengths(vs_ctx* c, int32_t* out) {
  if (!c || !out) return set_err(VS_ERR_INVALID_ARGUMENT, "NULL argument");
  std::memcpy(out, c->h_list_len.data(), sizeof(int32_t) * c->n_spots);
  return VS_OK;
}

vs_status vs_debug_philox(int64_t n, const uint32_t* ctr, const uint32_t* key, uint32_t* out) {
  if (n < 0 || (n > 0 && (!ctr || !key || !out))) return set_err(VS_ERR_INVALID_ARGUMENT, "bad arguments");
  if (n == 0) return VS_OK;
  vs_ctx* c = nullptr;
  uint4 *dc = nullptr, *dout = nullptr;
  CK(pool::alloc(&dc, sizeof(uint4) * n), "alloc");
  cudaError_t e = pool::alloc(&dout, sizeof(uint4) * n);
  if (e == cudaSuccess) e = cudaMemcpy(dc, ctr, sizeof(uint4) * n, cudaMemcpyHostToDevice);
  if (e == cudaSuccess) e = launch_philox(n, dc, make_uint2(key[0], key[1]), dout, nullptr);
  if (e == cudaSuccess) e = cudaMemcpy(out, dout, sizeof(uint4) * n, cudaMemcpyDeviceToHost);
  pool::release(dc);
  if (dout) pool::release(dout);
  if (e != cudaSuccess) return cuda_fail(c, e, "debug philox");
  return VS_OK;
}

}  // extern "C"
