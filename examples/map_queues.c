/* map_queues.c -- the C ABI used from plain C (no Python, no torch): one scheduling
 * decision of 4 queues on {CPU, GPU0, GPU1} with host buffers, plus a batch of epochs.
 *
 * Epoch 0 is DESIGN.md Appendix A case E ("EP-like": every queue 2000 ns on the CPU and
 * 100 ns on either GPU; EP goes to the GPUs): optimum (1, 1, 2, 2),
 * index 44, makespan 200. Epoch 1 is case F ("BT-like", [100, 350, 350] per queue; mostly
 * CPU, L1800-1807): (0, 0, 0, 1), index 1, makespan 350.
 * Then, on epoch 0: queue 0 pinned to the CPU (a SCHED_OFF queue, L838-845): the CPU carries
 * 2000 ns whatever the others do, so the optimum is 2000 and its lowest index keeps the other
 * queues off the CPU: (0, 1, 1, 1), index 13. And the SCHED_AUTO_STATIC policy (L1088-1116)
 * with every queue hinted compute-bound and a device profile favouring the GPUs equally sends
 * all four to GPU0 -- makespan 400, twice the optimum. Last, the resident mapper answers the
 * same decisions without a launch per call.
 *
 *   gcc -O2 -I include examples/map_queues.c -L paper_conf_cluster_ajipbf15_b200 -lmcl \
 *       -Wl,-rpath,$PWD/paper_conf_cluster_ajipbf15_b200 -o /tmp/map_queues
 */
#include <stdint.h>
#include <stdio.h>
#include <string.h>

#include "mcl.h"

int main(void) {
  enum { E = 2, Q = 4, D = 3 };
  uint64_t K[E][Q][D], X[E][Q][D];
  memset(X, 0, sizeof X);
  for (int q = 0; q < Q; ++q) {
    K[0][q][0] = 2000; K[0][q][1] = 100; K[0][q][2] = 100;
    K[1][q][0] = 100;  K[1][q][1] = 350; K[1][q][2] = 350;
  }
  mcl_config_t cfg;
  memset(&cfg, 0, sizeof cfg);
  cfg.device = 0;
  cfg.world = 1;
  mcl_mapper_t* h = NULL;
  mcl_status_t st = mcl_mapper_create(&cfg, &h);
  if (st != MCL_OK) {
    fprintf(stderr, "mcl_mapper_create: %s (%s)\n", mcl_status_string(st), mcl_last_error_string(NULL));
    return 1;
  }
  uint64_t index[E], makespan[E];
  uint8_t mapping[E][Q];
  st = mcl_map_queues(h, Q, D, E, &K[0][0][0], &X[0][0][0], index, &mapping[0][0], makespan);
  if (st != MCL_OK) {
    fprintf(stderr, "mcl_map_queues: %s (%s)\n", mcl_status_string(st), mcl_last_error_string(h));
    mcl_mapper_destroy(h);
    return 1;
  }
  const uint64_t want_index[E] = {44, 1}, want_ms[E] = {200, 350};
  int ok = 1;
  for (int e = 0; e < E; ++e) {
    printf("epoch %d: index %llu makespan %llu mapping", e, (unsigned long long)index[e],
           (unsigned long long)makespan[e]);
    for (int q = 0; q < Q; ++q) printf(" %u", mapping[e][q]);
    printf("\n");
    ok &= index[e] == want_index[e] && makespan[e] == want_ms[e];
  }
  /* constrained: queue 0 pinned to the CPU (one-bit eligible mask), the others free */
  uint16_t elig[Q] = {0x1, 0, 0, 0};
  mcl_constraints_t cons = {NULL, elig};
  uint64_t ci, cms;
  uint8_t cmap[Q];
  st = mcl_map_queues_constrained(h, Q, D, 1, &K[0][0][0], &X[0][0][0], &cons, &ci, cmap, &cms);
  printf("pinned queue 0: %s index %llu makespan %llu mapping %u %u %u %u\n", mcl_status_string(st),
         (unsigned long long)ci, (unsigned long long)cms, cmap[0], cmap[1], cmap[2], cmap[3]);
  ok &= st == MCL_OK && ci == 13 && cms == 2000;
  /* static hint policy vs the optimum: every queue compute-bound; class cost CPU 4, GPUs 1 */
  uint8_t hints[Q] = {0, 0, 0, 0}, smap[Q];
  const uint64_t score[1][D] = {{4, 1, 1}};
  uint64_t sms;
  st = mcl_static_mappings(h, Q, D, 1, hints, 1, &score[0][0], NULL, smap);
  if (st == MCL_OK) st = mcl_score_mappings(h, Q, D, 1, &K[0][0][0], &X[0][0][0], NULL, smap, &sms);
  printf("static policy: %s mapping %u %u %u %u makespan %llu\n", mcl_status_string(st), smap[0], smap[1],
         smap[2], smap[3], (unsigned long long)sms);
  ok &= st == MCL_OK && sms == 400 && smap[0] == 1 && smap[3] == 1;
  /* the resident mapper: one warp stays on the GPU and serves decisions from a pinned host
     mailbox (no launch per call); the same two epochs, then 1000 single decisions */
  st = mcl_resident_start(h, Q, D, E, 0);
  uint64_t ri[E], rms[E];
  uint8_t rmap[E][Q];
  if (st == MCL_OK) st = mcl_resident_map(h, E, &K[0][0][0], &X[0][0][0], ri, &rmap[0][0], rms);
  int rok = st == MCL_OK && ri[0] == 44 && rms[0] == 200 && ri[1] == 1 && rms[1] == 350;
  for (int i = 0; i < 1000 && st == MCL_OK; ++i) {
    st = mcl_resident_map(h, 1, &K[i & 1][0][0], &X[i & 1][0][0], ri, &rmap[0][0], rms);
    rok &= st == MCL_OK && ri[0] == want_index[i & 1] && rms[0] == want_ms[i & 1];
  }
  if (mcl_resident_stop(h) != MCL_OK) rok = 0;
  printf("resident: %s %s\n", mcl_status_string(st), rok ? "agrees" : "differs");
  ok &= rok;
  /* an entry >= 2^48 is a range error, reported, not silently wrapped */
  K[1][2][1] = (uint64_t)1 << 48;
  st = mcl_map_queues(h, Q, D, E, &K[0][0][0], &X[0][0][0], index, NULL, makespan);
  printf("entry 2^48: %s\n", mcl_status_string(st));
  ok &= st == MCL_E_RANGE;
  mcl_mapper_destroy(h);
  printf("%s\n", ok ? "OK" : "MISMATCH");
  return ok ? 0 : 2;
}
