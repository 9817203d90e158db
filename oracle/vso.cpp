// oracle/vso.cpp -- fp64 CPU ORACLE (test infrastructure, see vso.h header).
//
// Plain, slow, obviously-correct implementation of what the hot path
// computes.  Citations: "P:N" = line N of the paper text;
// "Rn" = reading n listed in DESIGN.md §3 (the paper is silent there).
//
// Build: g++ -O2 -std=c++17 -fopenmp -ffp-contract=off -fPIC -shared
//        (no -ffast-math; fp32 pose operations must be single IEEE ops).
#include "vso.h"

#include <algorithm>
#include <atomic>
#include <cmath>
#include <cstdio>
#include <cstring>
#include <new>
#include <string>
#include <vector>
#ifdef _OPENMP
#include <omp.h>
#endif

namespace {

thread_local std::string g_err;

vso_status fail(vso_status s, const char* msg) {
  g_err = msg;
  return s;
}

// ---------------------------------------------------------------------------
// Built-in atom-type table (R4, R5): sigma (A), epsilon (kcal/mol), HB role
// (0 none, 1 donor, 2 acceptor).  AMBER-parm99-like values.
// ---------------------------------------------------------------------------
const float kSigma[7] = {3.400f, 3.250f, 2.960f, 3.564f, 2.650f, 1.069f, 0.0f};
const float kEps[7] = {0.1094f, 0.170f, 0.210f, 0.250f, 0.0157f, 0.0157f, 0.0f};
const int kRole[7] = {0, 2, 2, 0, 0, 1, 0};
enum { ROLE_NONE = 0, ROLE_DONOR = 1, ROLE_ACCEPTOR = 2 };

// Philox stream tags (R23)
enum { TAG_INIT_ROT = 1, TAG_INIT_TRANS = 2, TAG_PARENT = 3, TAG_CROSS = 4, TAG_MUT = 5, TAG_LS = 6 };

struct Pose {
  float q[4];   // w, x, y, z
  float t[3];   // spot-relative translation (A)
  double score; // fp64 score
};

}  // namespace

struct vso_ctx {
  int n_rec = 0, n_lig = 0, n_spots = 0;
  std::vector<double> rec_xyz, rec_q;   // absolute receptor coordinates
  std::vector<int> rec_type;
  std::vector<float> lig_local;         // l_i = lig_xyz - centroid (fp32), [n_lig][3]
  std::vector<double> lig_q;
  std::vector<int> lig_type;
  std::vector<double> spot_xyz;
  // parameters
  double k, eps_r, rc, r2min, hb_eps, hb_r0;
  int dielectric;
  bool all_pairs;
  float T;                               // region half-width (fp32, R24)
  std::vector<double> sigma, eps, c12, c6;
  std::vector<int> role;
  double hb_C, hb_D;
  std::atomic<uint64_t> pairs{0};
  std::atomic<uint64_t> pairs_within{0};  // pairs inside the cutoff (instrumentation)
};

namespace {

bool finite3(const float* p, int64_t n) {
  for (int64_t i = 0; i < n; ++i)
    if (!std::isfinite(p[i])) return false;
  return true;
}

// ---------------------------------------------------------------------------
// Philox4x32-10 (Salmon et al., Random123; R23).  Counter-based: the stream
// for (seed, spot, individual, generation) needs no state.
// ---------------------------------------------------------------------------
void philox(const uint32_t ctr[4], const uint32_t key[2], uint32_t out[4]) {
  const uint32_t M0 = 0xD2511F53u, M1 = 0xCD9E8D57u;
  const uint32_t W0 = 0x9E3779B9u, W1 = 0xBB67AE85u;
  uint32_t c0 = ctr[0], c1 = ctr[1], c2 = ctr[2], c3 = ctr[3];
  uint32_t k0 = key[0], k1 = key[1];
  for (int round = 0; round < 10; ++round) {
    if (round > 0) { k0 += W0; k1 += W1; }
    uint64_t p0 = (uint64_t)M0 * c0;
    uint64_t p1 = (uint64_t)M1 * c2;
    uint32_t hi0 = (uint32_t)(p0 >> 32), lo0 = (uint32_t)p0;
    uint32_t hi1 = (uint32_t)(p1 >> 32), lo1 = (uint32_t)p1;
    uint32_t n0 = hi1 ^ c1 ^ k0;
    uint32_t n1 = lo1;
    uint32_t n2 = hi0 ^ c3 ^ k1;
    uint32_t n3 = lo0;
    c0 = n0; c1 = n1; c2 = n2; c3 = n3;
  }
  out[0] = c0; out[1] = c1; out[2] = c2; out[3] = c3;
}

// philox(i, s, g, tag, k) with key = (lo32(seed), hi32(seed))   (R23)
void stream(uint64_t seed, uint32_t i, uint32_t s, uint32_t g, uint32_t tag, uint32_t k, uint32_t w[4]) {
  uint32_t ctr[4] = {i, s, g, (tag << 24) | k};
  uint32_t key[2] = {(uint32_t)(seed & 0xFFFFFFFFu), (uint32_t)(seed >> 32)};
  philox(ctr, key, w);
}

// u01(w) = (w >> 8) * 2^-24 (exact);  v11 = 2*u01 - 1 (exact)   (R23)
float u01(uint32_t w) { return (float)(w >> 8) * (1.0f / 16777216.0f); }
float v11(uint32_t w) { return 2.0f * u01(w) - 1.0f; }

// ---------------------------------------------------------------------------
// fp32 pose operators, single IEEE ops in the written order (R24).
// volatile-free: compiled with -ffp-contract=off so no FMA is formed.
// ---------------------------------------------------------------------------
void normalize_q(float q[4]) {
  float n2 = ((q[0] * q[0] + q[1] * q[1]) + q[2] * q[2]) + q[3] * q[3];
  float n = std::sqrt(n2);
  for (int c = 0; c < 4; ++c) q[c] = q[c] / n;
}

// Hamilton product a (x) b
void hamilton(const float a[4], const float b[4], float o[4]) {
  float w = ((a[0] * b[0] - a[1] * b[1]) - a[2] * b[2]) - a[3] * b[3];
  float x = ((a[0] * b[1] + a[1] * b[0]) + a[2] * b[3]) - a[3] * b[2];
  float y = ((a[0] * b[2] - a[1] * b[3]) + a[2] * b[0]) + a[3] * b[1];
  float z = ((a[0] * b[3] + a[1] * b[2]) - a[2] * b[1]) + a[3] * b[0];
  o[0] = w; o[1] = x; o[2] = y; o[3] = z;
}

// uniform random rotation: rejection sampling in the 4-ball (R12)
void rand_quat(uint64_t seed, uint32_t i, uint32_t s, uint32_t g, float q[4]) {
  for (uint32_t k = 0; k < 64; ++k) {
    uint32_t w[4];
    stream(seed, i, s, g, TAG_INIT_ROT, k, w);
    float a = v11(w[0]), b = v11(w[1]), c = v11(w[2]), d = v11(w[3]);
    float n2 = ((a * a + b * b) + c * c) + d * d;
    if (n2 > 0.0f && n2 <= 1.0f) {
      float n = std::sqrt(n2);
      q[0] = a / n; q[1] = b / n; q[2] = c / n; q[3] = d / n;
      return;
    }
  }
  q[0] = 1.0f; q[1] = 0.0f; q[2] = 0.0f; q[3] = 0.0f;
}

// perturbation in the neighbourhood of a conformation: "moving, translating
// and/or rotating with respect to each spot" (R16)
void perturb(Pose& p, float dt, float dr, float T, uint64_t seed, uint32_t i, uint32_t s, uint32_t g,
             uint32_t tag, uint32_t k) {
  uint32_t a[4], b[4];
  stream(seed, i, s, g, tag, k, a);
  stream(seed, i, s, g, tag, k + 1, b);
  for (int c = 0; c < 3; ++c) {
    float m = dt * v11(a[c]);
    float t = p.t[c] + m;
    p.t[c] = std::min(std::max(t, -T), T);
  }
  float dq[4] = {1.0f, dr * v11(b[0]), dr * v11(b[1]), dr * v11(b[2])};
  float o[4];
  hamilton(dq, p.q, o);
  normalize_q(o);
  for (int c = 0; c < 4; ++c) p.q[c] = o[c];
}

// ---------------------------------------------------------------------------
// Scoring function (readings R1-R8), fp64, brute force over all
// receptor atoms.  Returns the score in kcal/mol.
// ---------------------------------------------------------------------------
// per-type LJ coefficients c12 = 2 sqrt(eps) sigma^6, c6 = 2 sqrt(eps) sigma^3 (R4), set in vso_create
double lj_c12(const vso_ctx* c, int t) { return c->c12[t]; }
double lj_c6(const vso_ctx* c, int t) { return c->c6[t]; }

double pair_energy(const vso_ctx* c, int ti, double qi, int tj, double qj, double r2) {
  // r^2 clamp (R7)
  if (r2 < c->r2min) r2 = c->r2min;
  double shift = 1.0;
  if (!c->all_pairs) {
    double rc2 = c->rc * c->rc;
    if (!(r2 < rc2)) return 0.0;               // cutoff (R6)
    double u = 1.0 - r2 / rc2;
    shift = u * u;                              // electrostatic shift (R6)
  }
  // electrostatics (R2, R3): distance-dependent eps(r) = 4r -> k qi qj / (4 r^2)
  double e_es;
  if (c->dielectric == 0)
    e_es = c->k * qi * qj / (4.0 * r2);
  else
    e_es = c->k * qi * qj / (c->eps_r * std::sqrt(r2));
  e_es *= shift;
  // Lennard-Jones 12-6 with geometric combining (R4):
  // 4 eps_ij [(sig_ij/r)^12 - (sig_ij/r)^6] = c12_i c12_j / r^12 - c6_i c6_j / r^6
  double r6 = r2 * r2 * r2;
  double r12 = r6 * r6;
  double e_vdw = lj_c12(c, ti) * lj_c12(c, tj) / r12 - lj_c6(c, ti) * lj_c6(c, tj) / r6;
  // hydrogen bond 12-10 (R5): w_ij = 1 iff one is a donor and the other an acceptor
  double e_hb = 0.0;
  int ri = c->role[ti], rj = c->role[tj];
  if ((ri == ROLE_DONOR && rj == ROLE_ACCEPTOR) || (ri == ROLE_ACCEPTOR && rj == ROLE_DONOR)) {
    // 12-10 well with minimum -hb_eps at r = hb_r0: C = 5 eps r0^12, D = 6 eps r0^10
    double C = c->hb_C, D = c->hb_D;
    double r10 = r6 * r2 * r2;
    e_hb = C / r12 - D / r10;
  }
  return e_es + e_vdw + e_hb;
}

// pose (s, q, t): x_i = c_s + t + R(q) l_i  (R11; homogeneous R, accepts non-unit q)
double score_pose(const vso_ctx* c, int s, const float qf[4], const float tf[3]) {
  double w = qf[0], x = qf[1], y = qf[2], z = qf[3];
  double s2 = 2.0 / (w * w + x * x + y * y + z * z);
  double R[3][3] = {
      {1.0 - s2 * (y * y + z * z), s2 * (x * y - w * z), s2 * (x * z + w * y)},
      {s2 * (x * y + w * z), 1.0 - s2 * (x * x + z * z), s2 * (y * z - w * x)},
      {s2 * (x * z - w * y), s2 * (y * z + w * x), 1.0 - s2 * (x * x + y * y)}};
  double total = 0.0;
  uint64_t within = 0;  // instrumentation: pairs inside the cutoff (all pairs in all-pairs mode)
  for (int i = 0; i < c->n_lig; ++i) {
    double l[3] = {c->lig_local[3 * i], c->lig_local[3 * i + 1], c->lig_local[3 * i + 2]};
    double xi[3];
    for (int a = 0; a < 3; ++a)
      xi[a] = c->spot_xyz[3 * s + a] + (double)tf[a] + (R[a][0] * l[0] + R[a][1] * l[1] + R[a][2] * l[2]);
    for (int j = 0; j < c->n_rec; ++j) {
      double dx = xi[0] - c->rec_xyz[3 * j], dy = xi[1] - c->rec_xyz[3 * j + 1], dz = xi[2] - c->rec_xyz[3 * j + 2];
      double r2 = dx * dx + dy * dy + dz * dz;
      total += pair_energy(c, c->lig_type[i], c->lig_q[i], c->rec_type[j], c->rec_q[j], r2);
      within += c->all_pairs || std::max(r2, c->r2min) < c->rc * c->rc;
    }
  }
  const_cast<vso_ctx*>(c)->pairs.fetch_add((uint64_t)c->n_lig * (uint64_t)c->n_rec, std::memory_order_relaxed);
  const_cast<vso_ctx*>(c)->pairs_within.fetch_add(within, std::memory_order_relaxed);
  return total;
}

// Decisions that the scores take (Improve's accept, the sorts of Select/Include) are made on the scores
// rounded to fp32, the precision of the kernel (R26); the scores themselves stay fp64.
float dec(double s) { return (float)s; }

bool less_score_index(double sa, int ia, double sb, int ib) {
  return dec(sa) < dec(sb) || (dec(sa) == dec(sb) && ia < ib);
}

// ---------------------------------------------------------------------------
// Algorithm 1, per spot.
// ---------------------------------------------------------------------------
struct MH {
  const vso_ctx* c;
  vso_mh_params mp;
  uint64_t seed;
  int s;  // global spot id (keys the RNG)
  int m;  // number of elements improved

  // Initialize(S): random population, scored; improved when f > 0
  // (M2: "all the elements are improved after they have been generated
  // initially"); then ordered by (score, index).
  void initialize(std::vector<Pose>& S) {
    int P = mp.population;
    S.resize(P);
    for (int i = 0; i < P; ++i) {
      init_pose(i, S[i]);
      S[i].score = score_pose(c, s, S[i].q, S[i].t);
    }
    if (mp.improve_frac > 0.0f) improve(S, 0);
    sort_by_score(S);
  }

  void init_pose(int i, Pose& p) {
    rand_quat(seed, i, s, 0, p.q);
    uint32_t w[4];
    stream(seed, i, s, 0, TAG_INIT_TRANS, 0, w);
    for (int a = 0; a < 3; ++a) p.t[a] = c->T * v11(w[a]);
  }

  // End(S): fixed number of generations (R20)
  bool end(int g) const { return g > mp.generations; }

  // Select(S, Ssel): 100 % of S selected (T4); the parents of child j
  // are two binary tournaments on ranks (R13).  S is sorted: rank = index.
  void select(int g, int j, int& p1, int& p2) const {
    uint32_t P = (uint32_t)mp.population;
    uint32_t w[4];
    stream(seed, j, s, g, TAG_PARENT, 0, w);
    p1 = (int)std::min(w[0] % P, w[1] % P);
    p2 = (int)std::min(w[2] % P, w[3] % P);
    if (p2 == p1) p2 = (p1 + 1) % (int)P;
  }

  // Combine(Ssel, Scom): blend crossover + mutation (R14, R15)
  void combine_child(const std::vector<Pose>& S, int g, int j, Pose& out) const {
    int p1, p2;
    select(g, j, p1, p2);
    const Pose& A = S[p1];
    const Pose& B = S[p2];
    uint32_t w[4];
    stream(seed, j, s, g, TAG_CROSS, 0, w);
    float alpha = u01(w[0]);
    float beta = 1.0f - alpha;
    for (int a = 0; a < 3; ++a) {
      float d = B.t[a] - A.t[a];
      float mm = alpha * d;
      out.t[a] = A.t[a] + mm;
    }
    float dot = ((A.q[0] * B.q[0] + A.q[1] * B.q[1]) + A.q[2] * B.q[2]) + A.q[3] * B.q[3];
    float q2[4];
    for (int a = 0; a < 4; ++a) q2[a] = dot < 0.0f ? -B.q[a] : B.q[a];
    for (int a = 0; a < 4; ++a) out.q[a] = beta * A.q[a] + alpha * q2[a];
    normalize_q(out.q);
    stream(seed, j, s, g, TAG_MUT, 0, w);
    if (u01(w[0]) < mp.p_mut) perturb(out, mp.mut_trans, mp.mut_rot, c->T, seed, j, s, g, TAG_MUT, 1);
  }

  void combine(const std::vector<Pose>& S, int g, std::vector<Pose>& Scom) const {
    int P = mp.population;
    Scom.resize(P);
    for (int j = 0; j < P; ++j) combine_child(S, g, j, Scom[j]);
  }

  // Improve(Scom): local search in the neighbourhood of the best m
  // elements (R16, R17): L steps, strict <.  With K = ls_neighbours proposals
  // per step the best of the K replaces the element if it is strictly better
  // (lowest k on ties; K = 1 is first-improvement hill climbing).
  void improve(std::vector<Pose>& X, int g) const {
    int P = (int)X.size();
    std::vector<double> sc(P);
    for (int i = 0; i < P; ++i) sc[i] = X[i].score;
    std::vector<int> J(m);
    vso_select_improve(sc.data(), P, m, J.data());
    const int K = mp.ls_neighbours;
    for (int l = 0; l < mp.ls_steps; ++l) {
      for (int j : J) {
        Pose best = X[j];
        for (int k = 0; k < K; ++k) {
          Pose cand = X[j];
          perturb(cand, mp.ls_trans, mp.ls_rot, c->T, seed, j, s, g, TAG_LS, 2 * (l * K + k));
          cand.score = score_pose(c, s, cand.q, cand.t);
          if (dec(cand.score) < dec(best.score)) best = cand;
        }
        X[j] = best;
      }
    }
  }

  // Include(Scom, S): best P of S and Scom (R19)
  void include(std::vector<Pose>& S, const std::vector<Pose>& Scom) const {
    int P = mp.population;
    std::vector<double> sS(P), sC(P);
    for (int i = 0; i < P; ++i) { sS[i] = S[i].score; sC[i] = Scom[i].score; }
    std::vector<int> origin(P);
    vso_include(sS.data(), sC.data(), P, origin.data());
    std::vector<Pose> next(P);
    for (int k = 0; k < P; ++k) next[k] = origin[k] < P ? S[origin[k]] : Scom[origin[k] - P];
    S.swap(next);
  }

  static void sort_by_score(std::vector<Pose>& S) {
    std::stable_sort(S.begin(), S.end(), [](const Pose& a, const Pose& b) { return dec(a.score) < dec(b.score); });
  }

  Pose run() {
    std::vector<Pose> S, Scom;
    initialize(S);
    for (int g = 1; !end(g); ++g) {
      combine(S, g, Scom);                       // Select + Combine
      for (auto& p : Scom) p.score = score_pose(c, s, p.q, p.t);
      if (mp.improve_frac > 0.0f) improve(Scom, g);
      include(S, Scom);
    }
    return S[0];
  }
};

vso_status check_mh(const vso_mh_params* mp) {
  if (!mp) return fail(VSO_ERR_INVALID_ARGUMENT, "mh params: NULL");
  if (mp->population < 1 || mp->population > 2048) return fail(VSO_ERR_INVALID_ARGUMENT, "population must be in [1, 2048]");
  if (mp->generations < 0) return fail(VSO_ERR_INVALID_ARGUMENT, "generations must be >= 0");
  if (mp->generations > 0 && mp->population < 2) return fail(VSO_ERR_INVALID_ARGUMENT, "population must be >= 2 when generations > 0");
  if (mp->ls_steps < 0) return fail(VSO_ERR_INVALID_ARGUMENT, "ls_steps must be >= 0");
  if (mp->ls_neighbours < 1 || mp->ls_neighbours > 64) return fail(VSO_ERR_INVALID_ARGUMENT, "ls_neighbours must be in [1, 64]");
  // LS counter word (TAG_LS << 24) | (2 (l K + k) + 1) stays below 2^24 (R23)
  if ((long long)mp->ls_steps * mp->ls_neighbours > (1ll << 23))
    return fail(VSO_ERR_INVALID_ARGUMENT, "ls_steps x ls_neighbours must be <= 2^23");
  if (!(mp->improve_frac >= 0.0f && mp->improve_frac <= 1.0f)) return fail(VSO_ERR_INVALID_ARGUMENT, "improve_frac must be in [0, 1]");
  if (!(mp->p_mut >= 0.0f && mp->p_mut <= 1.0f)) return fail(VSO_ERR_INVALID_ARGUMENT, "p_mut must be in [0, 1]");
  const float st[4] = {mp->mut_trans, mp->mut_rot, mp->ls_trans, mp->ls_rot};
  for (float v : st)
    if (!(std::isfinite(v) && v >= 0.0f)) return fail(VSO_ERR_INVALID_ARGUMENT, "step sizes must be finite and >= 0");
  return VSO_OK;
}

}  // namespace

extern "C" {

void vso_score_params_default(vso_score_params* o) {
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
}

// Table 4 + readings R15-R18, R21
vso_status vso_mh_preset(int m, vso_mh_params* o) {
  if (!o) return fail(VSO_ERR_INVALID_ARGUMENT, "out: NULL");
  if (m < 1 || m > 4) return fail(VSO_ERR_INVALID_ARGUMENT, "preset must be 1..4");
  o->population = (m == 4) ? 1024 : 64;
  o->generations = (m == 4) ? 0 : 50;
  o->ls_steps = (m == 1) ? 0 : 8;
  o->improve_frac = (m == 1) ? 0.0f : (m == 3 ? 0.2f : 1.0f);
  o->p_mut = 0.1f;
  o->mut_trans = 1.0f;
  o->mut_rot = 0.25f;
  o->ls_trans = 0.5f;
  o->ls_rot = 0.10f;
  o->ls_neighbours = 1;
  return VSO_OK;
}

vso_status vso_create(const float* rec_xyz, const float* rec_q, const int32_t* rec_type, int32_t n_rec,
                      const float* lig_xyz, const float* lig_q, const int32_t* lig_type, int32_t n_lig,
                      const float* spot_xyz, int32_t n_spots, const vso_score_params* sp_in,
                      int32_t /*cuda_device*/, vso_ctx** out) {
  if (!out) return fail(VSO_ERR_INVALID_ARGUMENT, "out: NULL");
  *out = nullptr;
  if (!rec_xyz || !rec_q || !rec_type || !lig_xyz || !lig_q || !lig_type || !spot_xyz)
    return fail(VSO_ERR_INVALID_ARGUMENT, "NULL input array");
  if (n_rec < 1 || n_lig < 1 || n_lig > 256 || n_spots < 1)
    return fail(VSO_ERR_INVALID_ARGUMENT, "need n_rec >= 1, 1 <= n_lig <= 256, n_spots >= 1");
  vso_score_params sp;
  if (sp_in) sp = *sp_in; else vso_score_params_default(&sp);
  if (!(std::isfinite(sp.coulomb_k)) || (sp.dielectric != 0 && sp.dielectric != 1) ||
      (sp.dielectric == 1 && !(sp.eps_r > 0.0f && std::isfinite(sp.eps_r))) ||
      !(sp.region_half_width > 0.0f && std::isfinite(sp.region_half_width)) ||
      !(sp.hb_eps >= 0.0f && std::isfinite(sp.hb_eps)) || !(sp.hb_r0 > 0.0f && std::isfinite(sp.hb_r0)) ||
      !(sp.r2_min > 0.0f && std::isfinite(sp.r2_min)) || std::isnan(sp.cutoff))
    return fail(VSO_ERR_INVALID_ARGUMENT, "invalid score params");
  if (sp.n_types < 0 || (sp.n_types > 0 && (!sp.type_sigma || !sp.type_eps || !sp.type_hb_role)) || sp.n_types > 64)
    return fail(VSO_ERR_INVALID_ARGUMENT, "invalid type table");
  if (!finite3(rec_xyz, 3 * (int64_t)n_rec) || !finite3(rec_q, n_rec) || !finite3(lig_xyz, 3 * (int64_t)n_lig) ||
      !finite3(lig_q, n_lig) || !finite3(spot_xyz, 3 * (int64_t)n_spots))
    return fail(VSO_ERR_INVALID_ARGUMENT, "non-finite input");
  vso_ctx* c = new (std::nothrow) vso_ctx;
  if (!c) return fail(VSO_ERR_OUT_OF_MEMORY, "out of host memory");
  int nt = sp.n_types > 0 ? sp.n_types : 7;
  for (int t = 0; t < nt; ++t) {
    float sg = sp.n_types > 0 ? sp.type_sigma[t] : kSigma[t];
    float ep = sp.n_types > 0 ? sp.type_eps[t] : kEps[t];
    int rl = sp.n_types > 0 ? sp.type_hb_role[t] : kRole[t];
    if (!(sg >= 0.0f && std::isfinite(sg)) || !(ep >= 0.0f && std::isfinite(ep)) || rl < 0 || rl > 2) {
      delete c;
      return fail(VSO_ERR_INVALID_ARGUMENT, "invalid type table entry");
    }
    c->sigma.push_back(sg);
    c->eps.push_back(ep);
    c->role.push_back(rl);
    c->c12.push_back(2.0 * std::sqrt((double)ep) * std::pow((double)sg, 6));
    c->c6.push_back(2.0 * std::sqrt((double)ep) * std::pow((double)sg, 3));
  }
  for (int i = 0; i < n_rec; ++i)
    if (rec_type[i] < 0 || rec_type[i] >= nt) { delete c; return fail(VSO_ERR_INVALID_ARGUMENT, "receptor type id out of range"); }
  for (int i = 0; i < n_lig; ++i)
    if (lig_type[i] < 0 || lig_type[i] >= nt) { delete c; return fail(VSO_ERR_INVALID_ARGUMENT, "ligand type id out of range"); }
  c->n_rec = n_rec; c->n_lig = n_lig; c->n_spots = n_spots;
  c->rec_xyz.assign(rec_xyz, rec_xyz + 3 * (size_t)n_rec);
  c->rec_q.assign(rec_q, rec_q + n_rec);
  c->rec_type.assign(rec_type, rec_type + n_rec);
  c->lig_q.assign(lig_q, lig_q + n_lig);
  c->lig_type.assign(lig_type, lig_type + n_lig);
  c->spot_xyz.assign(spot_xyz, spot_xyz + 3 * (size_t)n_spots);
  // ligand centred on its centroid: centroid in fp64, rounded to fp32 once (R11)
  float cen[3];
  for (int a = 0; a < 3; ++a) {
    double acc = 0.0;
    for (int i = 0; i < n_lig; ++i) acc += lig_xyz[3 * i + a];
    cen[a] = (float)(acc / n_lig);
  }
  c->lig_local.resize(3 * (size_t)n_lig);
  for (int i = 0; i < n_lig; ++i)
    for (int a = 0; a < 3; ++a) c->lig_local[3 * i + a] = lig_xyz[3 * i + a] - cen[a];
  c->k = sp.coulomb_k;
  c->dielectric = sp.dielectric;
  c->eps_r = sp.eps_r;
  c->all_pairs = !(sp.cutoff > 0.0f) || std::isinf(sp.cutoff);
  c->rc = c->all_pairs ? INFINITY : (double)sp.cutoff;
  c->r2min = sp.r2_min;
  c->hb_eps = sp.hb_eps;
  c->hb_r0 = sp.hb_r0;
  c->T = sp.region_half_width;
  c->hb_C = 5.0 * c->hb_eps * std::pow(c->hb_r0, 12);
  c->hb_D = 6.0 * c->hb_eps * std::pow(c->hb_r0, 10);
  *out = c;
  return VSO_OK;
}

static vso_status score_common(vso_ctx* c, int64_t n, const int32_t* spot, const float* q, const float* t,
                               float* outf, double* outd) {
  if (!c) return fail(VSO_ERR_INVALID_ARGUMENT, "ctx: NULL");
  if (n < 0) return fail(VSO_ERR_INVALID_ARGUMENT, "n must be >= 0");
  if (n == 0) return VSO_OK;
  if (!spot || !q || !t || (!outf && !outd)) return fail(VSO_ERR_INVALID_ARGUMENT, "NULL pose array");
  for (int64_t p = 0; p < n; ++p) {
    if (spot[p] < 0 || spot[p] >= c->n_spots) return fail(VSO_ERR_INVALID_ARGUMENT, "spot id out of range");
    for (int a = 0; a < 4; ++a)
      if (!std::isfinite(q[4 * p + a])) return fail(VSO_ERR_INVALID_ARGUMENT, "non-finite quaternion");
    for (int a = 0; a < 3; ++a)
      if (!std::isfinite(t[3 * p + a])) return fail(VSO_ERR_INVALID_ARGUMENT, "non-finite translation");
    if (q[4 * p] == 0.0f && q[4 * p + 1] == 0.0f && q[4 * p + 2] == 0.0f && q[4 * p + 3] == 0.0f)
      return fail(VSO_ERR_ZERO_QUATERNION, "zero quaternion");
    if (!c->all_pairs)
      for (int a = 0; a < 3; ++a)
        if (std::fabs(t[3 * p + a]) > c->T) return fail(VSO_ERR_POSE_OUT_OF_REGION, "translation outside the spot region");
  }
#pragma omp parallel for schedule(dynamic, 1)
  for (int64_t p = 0; p < n; ++p) {
    double e = score_pose(c, spot[p], q + 4 * p, t + 3 * p);
    if (outf) outf[p] = (float)e;
    if (outd) outd[p] = e;
  }
  return VSO_OK;
}

vso_status vso_score_poses(vso_ctx* c, int64_t n, const int32_t* spot, const float* q, const float* t, float* out) {
  return score_common(c, n, spot, q, t, out, nullptr);
}

vso_status vso_score_poses_d(vso_ctx* c, int64_t n, const int32_t* spot, const float* q, const float* t, double* out) {
  return score_common(c, n, spot, q, t, nullptr, out);
}

static vso_status run_common(vso_ctx* c, const vso_mh_params* mp, uint64_t seed, int32_t n_sel,
                             const int32_t* spot_ids, float* best_pose, float* best_f, double* best_d) {
  if (!c) return fail(VSO_ERR_INVALID_ARGUMENT, "ctx: NULL");
  vso_status st = check_mh(mp);
  if (st != VSO_OK) return st;
  if (n_sel < 0 || (n_sel == 0 && spot_ids)) return fail(VSO_ERR_INVALID_ARGUMENT, "n_sel must be >= 1 with spot_ids");
  int ns = spot_ids ? n_sel : c->n_spots;
  if (!spot_ids && n_sel != 0 && n_sel != c->n_spots)
    return fail(VSO_ERR_INVALID_ARGUMENT, "n_sel must be 0 or n_spots when spot_ids is NULL");
  if (!best_pose || (!best_f && !best_d)) return fail(VSO_ERR_INVALID_ARGUMENT, "NULL output");
  if (spot_ids)
    for (int k = 0; k < ns; ++k)
      if (spot_ids[k] < 0 || spot_ids[k] >= c->n_spots) return fail(VSO_ERR_INVALID_ARGUMENT, "spot id out of range");
  int m = vso_improve_count(mp);
#pragma omp parallel for schedule(dynamic, 1)
  for (int k = 0; k < ns; ++k) {
    MH mh{c, *mp, seed, spot_ids ? spot_ids[k] : k, m};
    Pose best = mh.run();
    for (int a = 0; a < 4; ++a) best_pose[7 * k + a] = best.q[a];
    for (int a = 0; a < 3; ++a) best_pose[7 * k + 4 + a] = best.t[a];
    if (best_f) best_f[k] = (float)best.score;
    if (best_d) best_d[k] = best.score;
  }
  return VSO_OK;
}

vso_status vso_run(vso_ctx* c, const vso_mh_params* mp, uint64_t seed, int32_t n_sel, const int32_t* spot_ids,
                   float* best_pose_out, float* best_score_out) {
  return run_common(c, mp, seed, n_sel, spot_ids, best_pose_out, best_score_out, nullptr);
}

vso_status vso_run_d(vso_ctx* c, const vso_mh_params* mp, uint64_t seed, int32_t n_sel, const int32_t* spot_ids,
                     float* best_pose_out, double* best_score_out) {
  return run_common(c, mp, seed, n_sel, spot_ids, best_pose_out, nullptr, best_score_out);
}

void vso_destroy(vso_ctx* c) { delete c; }
const char* vso_last_error(void) { return g_err.c_str(); }
int vso_abi_version(void) { return 2; }

void vso_set_threads(int n) {
#ifdef _OPENMP
  omp_set_num_threads(n > 0 ? n : omp_get_num_procs());
#else
  (void)n;
#endif
}

int vso_get_threads(void) {
#ifdef _OPENMP
  return omp_get_max_threads();
#else
  return 1;
#endif
}

void vso_philox4x32_10(const uint32_t ctr[4], const uint32_t key[2], uint32_t out[4]) { philox(ctr, key, out); }
float vso_u01(uint32_t w) { return u01(w); }
float vso_v11(uint32_t w) { return v11(w); }

double vso_score_one(const vso_ctx* c, int32_t spot, const float q[4], const float t[3]) {
  return score_pose(c, spot, q, t);
}

void vso_ligand_local(const vso_ctx* c, float* out) {
  std::memcpy(out, c->lig_local.data(), sizeof(float) * c->lig_local.size());
}

uint64_t vso_pairs_evaluated(const vso_ctx* c) { return c->pairs.load(); }
uint64_t vso_pairs_within(const vso_ctx* c) { return c->pairs_within.load(); }

static void to_pose(const float in[7], Pose& p) {
  for (int a = 0; a < 4; ++a) p.q[a] = in[a];
  for (int a = 0; a < 3; ++a) p.t[a] = in[4 + a];
  p.score = 0.0;
}
static void from_pose(const Pose& p, float out[7]) {
  for (int a = 0; a < 4; ++a) out[a] = p.q[a];
  for (int a = 0; a < 3; ++a) out[4 + a] = p.t[a];
}

void vso_init_pose(const vso_ctx* c, uint64_t seed, int32_t spot, int32_t i, float out[7]) {
  vso_mh_params mp;
  vso_mh_preset(1, &mp);
  MH mh{c, mp, seed, spot, 1};
  Pose p;
  mh.init_pose(i, p);
  from_pose(p, out);
}

void vso_combine_child(const vso_ctx* c, const vso_mh_params* mp, uint64_t seed, int32_t spot, int32_t g,
                       int32_t j, const float* S_sorted, float out[7]) {
  MH mh{c, *mp, seed, spot, 1};
  std::vector<Pose> S(mp->population);
  for (int i = 0; i < mp->population; ++i) to_pose(S_sorted + 7 * i, S[i]);
  Pose o;
  mh.combine_child(S, g, j, o);
  from_pose(o, out);
}

void vso_select_parents(const vso_mh_params* mp, uint64_t seed, int32_t spot, int32_t g, int32_t j,
                        int32_t* p1_out, int32_t* p2_out) {
  MH mh{nullptr, *mp, seed, spot, 1};
  int p1, p2;
  mh.select(g, j, p1, p2);
  *p1_out = p1;
  *p2_out = p2;
}

void vso_ls_proposal(const vso_ctx* c, const vso_mh_params* mp, uint64_t seed, int32_t spot, int32_t g,
                     int32_t l, int32_t j, const float in[7], float out[7]) {
  vso_ls_proposal_k(c, mp, seed, spot, g, l, 0, j, in, out);
}

void vso_ls_proposal_k(const vso_ctx* c, const vso_mh_params* mp, uint64_t seed, int32_t spot, int32_t g,
                       int32_t l, int32_t k, int32_t j, const float in[7], float out[7]) {
  Pose p;
  to_pose(in, p);
  perturb(p, mp->ls_trans, mp->ls_rot, c->T, seed, j, spot, g, TAG_LS, 2 * (l * mp->ls_neighbours + k));
  from_pose(p, out);
}

// m = clamp(round-half-up(f * P), 1, P), f used as its fp32 value (R17)
int32_t vso_improve_count(const vso_mh_params* mp) {
  long long m = std::llround((double)mp->improve_frac * (double)mp->population);
  if (m < 1) m = 1;
  if (m > mp->population) m = mp->population;
  return (int32_t)m;
}

void vso_select_improve(const double* scores, int32_t P, int32_t m, int32_t* J) {
  std::vector<int> idx(P);
  for (int i = 0; i < P; ++i) idx[i] = i;
  std::sort(idx.begin(), idx.end(), [&](int a, int b) { return less_score_index(scores[a], a, scores[b], b); });
  for (int k = 0; k < m; ++k) J[k] = idx[k];
}

void vso_include(const double* sS, const double* sC, int32_t P, int32_t* origin) {
  std::vector<int> idx(2 * P);
  for (int i = 0; i < 2 * P; ++i) idx[i] = i;
  auto sc = [&](int i) { return i < P ? sS[i] : sC[i - P]; };
  std::stable_sort(idx.begin(), idx.end(), [&](int a, int b) { return dec(sc(a)) < dec(sc(b)); });
  for (int k = 0; k < P; ++k) origin[k] = idx[k];
}

}  // extern "C"
