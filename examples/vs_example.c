/* examples/vs_example.c -- the C ABI used directly from C (no Python):
 * a synthetic receptor / ligand, one batch of poses scored, one M3 run.
 *
 * build: gcc -O2 -I include examples/vs_example.c -L paper_conf_ppopp_imbernoncg16_b200 -lvs \
 *            -Wl,-rpath,$PWD/paper_conf_ppopp_imbernoncg16_b200 -lm -o vs_example
 */
#include <math.h>
#include <stdio.h>
#include <stdlib.h>

#include "vs.h"

static float frand(unsigned* s) {
  *s = *s * 1664525u + 1013904223u;
  return (float)(*s >> 8) / 16777216.0f;
}

int main(void) {
  enum { NREC = 2000, NLIG = 24, NSPOT = 8, NPOSE = 64 };
  static float rec_xyz[NREC * 3], rec_q[NREC], lig_xyz[NLIG * 3], lig_q[NLIG], spots[NSPOT * 3];
  static int32_t rec_t[NREC], lig_t[NLIG];
  unsigned s = 12345u;
  /* receptor: random atoms in a 16 A ball; ligand: 24 atoms in a 4 A ball; spots on the surface */
  for (int i = 0; i < NREC; ++i) {
    float x, y, z;
    do { x = 2 * frand(&s) - 1; y = 2 * frand(&s) - 1; z = 2 * frand(&s) - 1; } while (x * x + y * y + z * z > 1);
    rec_xyz[3 * i] = 16 * x; rec_xyz[3 * i + 1] = 16 * y; rec_xyz[3 * i + 2] = 16 * z;
    rec_q[i] = 0.4f * (frand(&s) - 0.5f);
    rec_t[i] = (int32_t)(frand(&s) * 6);      /* C N O S H HD */
  }
  for (int i = 0; i < NLIG; ++i) {
    lig_xyz[3 * i] = 4 * (frand(&s) - 0.5f); lig_xyz[3 * i + 1] = 4 * (frand(&s) - 0.5f);
    lig_xyz[3 * i + 2] = 4 * (frand(&s) - 0.5f);
    lig_q[i] = 0.4f * (frand(&s) - 0.5f);
    lig_t[i] = (int32_t)(frand(&s) * 6);
  }
  for (int k = 0; k < NSPOT; ++k) {
    float a = 6.2831853f * k / NSPOT;
    spots[3 * k] = 17 * cosf(a); spots[3 * k + 1] = 17 * sinf(a); spots[3 * k + 2] = 0;
  }
  vs_score_params sp;
  vs_score_params_default(&sp);
  vs_ctx* ctx = NULL;
  vs_status st = vs_create(rec_xyz, rec_q, rec_t, NREC, lig_xyz, lig_q, lig_t, NLIG, spots, NSPOT, &sp, 0, &ctx);
  if (st != VS_OK) { fprintf(stderr, "vs_create: %d %s\n", st, vs_last_error()); return 1; }

  static int32_t pspot[NPOSE];
  static float q[NPOSE * 4], t[NPOSE * 3], score[NPOSE];
  for (int p = 0; p < NPOSE; ++p) {
    pspot[p] = p % NSPOT;
    q[4 * p] = 1; q[4 * p + 1] = frand(&s) - 0.5f; q[4 * p + 2] = frand(&s) - 0.5f; q[4 * p + 3] = 0;
    for (int a = 0; a < 3; ++a) t[3 * p + a] = 3 * (2 * frand(&s) - 1);
  }
  st = vs_score_poses(ctx, NPOSE, pspot, q, t, score);
  if (st != VS_OK) { fprintf(stderr, "vs_score_poses: %d %s\n", st, vs_last_error()); return 1; }
  printf("score[0..3] = %.4f %.4f %.4f %.4f kcal/mol\n", score[0], score[1], score[2], score[3]);

  vs_mh_params mp;
  vs_mh_preset(3, &mp);
  mp.generations = 10;
  static float best_pose[NSPOT * 7], best[NSPOT];
  st = vs_run(ctx, &mp, 42, 0, NULL, best_pose, best);
  if (st != VS_OK) { fprintf(stderr, "vs_run: %d %s\n", st, vs_last_error()); return 1; }
  for (int k = 0; k < NSPOT; ++k) printf("spot %d best %.4f kcal/mol\n", k, best[k]);
  vs_stats stats;
  vs_get_stats(ctx, &stats);
  printf("kernels %llu, poses scored %llu, pairs %llu\n", (unsigned long long)stats.kernel_launches,
         (unsigned long long)stats.poses_scored, (unsigned long long)stats.pairs);
  vs_destroy(ctx);
  return 0;
}
