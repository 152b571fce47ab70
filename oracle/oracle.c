/*
 * oracle/oracle.c -- TEST INFRASTRUCTURE ONLY.
 *
 * A plain, slow, obviously-correct CPU brute force of MultiCL's device-mapper search
 * (Aji, Pena, Balaji, Feng, "Automatic Command Queue Scheduling for Task-Parallel
 * Workloads in OpenCL", IEEE CLUSTER 2015). It exists only so that tests/, bench.py's
 * cpu_baseline / --impl reference leg and __graft_entry__.smoke() can check and time the
 * CUDA product path. The product library never links, loads or calls this file, and this
 * file includes nothing from the product (no shared headers, helpers or tables).
 *
 * What it computes (SS V.A "Device Mapper": "determine the ideal
 * queue-device mapping that minimizes the concurrent execution time"; PAPER.md L2106-2118,
 * SS VI.B.1 summary: "computes the aggregate cost metric from the data transfer and kernel
 * execution costs"), for every epoch e independently:
 *
 *   C[q][d]   = K[q][d] + X[q][d]                     aggregate cost, integer ns
 *   digits(m) = (d_0 .. d_{Q-1}),  m = sum_q d_q * D^(Q-1-q)   queue 0 most significant
 *   L_d(m)    = sum over queues q with d_q == d of C[q][d]      (0 for an idle device)
 *   ms(m)     = max_d L_d(m)                          "concurrent execution time"
 *   m*        = the smallest m with ms(m) == min over all m' of ms(m')
 *
 * Readings of silent/garbled points (DESIGN.md "Readings" R1-R13): queues sharing a device
 * serialise (sum), distinct devices run concurrently (max); ties go to the lowest index
 * (BASELINE.json north_star); the search space is all D^Q tuples ("3^4" / "3^2" at
 * PAPER.md L1736-1738, L2229-2233 are 3^4 = 81 and 3^2 = 9 with flattened superscripts).
 *
 * Method: enumerate m = lo .. hi-1 in increasing order with an odometer over the digits,
 * recompute every device load from zero for every mapping, take the max, and keep the
 * first strict minimum. Threads (pthreads) take contiguous sub-ranges (or whole epochs);
 * the host merges their (ms, m) results lexicographically. No blocking, no factoring, no
 * pruning: every mapping is scored exactly as the definition reads.
 */
#include <pthread.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#define ORACLE_MAX_Q 32
#define ORACLE_MAX_D 16
#define ORACLE_ENTRY_LIMIT (1ULL << 48) /* DESIGN.md reading R10: entries < 2^48 */

/* status codes (same meaning as documented in DESIGN.md, defined independently here) */
#define ORACLE_OK 0
#define ORACLE_E_INVAL (-1)
#define ORACLE_E_RANGE (-2)

typedef struct {
  uint32_t Q, D;
  const uint64_t *K, *X; /* this epoch's [Q][D] tables */
  const uint64_t *base;  /* this epoch's [D] pre-existing device loads, or NULL (all 0) */
  const uint16_t *elig;  /* this epoch's [Q] eligible-device bit masks (0 = any), or NULL */
  uint64_t lo, hi;       /* mapping-index range [lo, hi) */
  uint64_t best_ms, best_m;
  int found;
} oracle_range_job;

/* Score mappings lo..hi-1 of one epoch. */
static void oracle_scan_range(oracle_range_job *job) {
  const uint32_t Q = job->Q, D = job->D;
  uint32_t digit[ORACLE_MAX_Q];
  uint64_t load[ORACLE_MAX_D];
  uint64_t m = job->lo;
  /* decode the first index into base-D digits, queue 0 most significant */
  uint64_t rest = m;
  for (int q = (int)Q - 1; q >= 0; --q) {
    digit[q] = (uint32_t)(rest % D);
    rest /= D;
  }
  job->found = 0;
  job->best_ms = 0;
  job->best_m = 0;
  for (; m < job->hi; ++m) {
    /* constrained variant (R11): a mapping that places a queue on a device
       outside its eligible set is not a candidate (SCHED_OFF queues are "statically
       mapped to the chosen device") */
    int feasible = 1;
    if (job->elig)
      for (uint32_t q = 0; q < Q; ++q)
        if (job->elig[q] != 0 && !((job->elig[q] >> digit[q]) & 1u)) feasible = 0;
    /* per-device loads: the pre-existing load of the device (0 without base loads),
       then every queue placed there -- queues on one device serialise (sum) */
    for (uint32_t d = 0; d < D; ++d) load[d] = job->base ? job->base[d] : 0;
    for (uint32_t q = 0; q < Q; ++q) {
      uint32_t d = digit[q];
      load[d] += job->K[q * D + d] + job->X[q * D + d]; /* aggregate cost C = K + X */
    }
    /* distinct devices run concurrently: makespan = max over devices */
    uint64_t ms = 0;
    for (uint32_t d = 0; d < D; ++d)
      if (load[d] > ms) ms = load[d];
    /* first strict minimum in increasing index order = lowest index among ties */
    if (feasible && (!job->found || ms < job->best_ms)) {
      job->found = 1;
      job->best_ms = ms;
      job->best_m = m;
    }
    /* odometer: increment the least significant digit (queue Q-1) with carry */
    for (int q = (int)Q - 1; q >= 0; --q) {
      if (++digit[q] < D) break;
      digit[q] = 0;
    }
  }
}

static void *oracle_thread_main(void *arg) {
  oracle_range_job *jobs = (oracle_range_job *)arg;
  /* a thread's job list is terminated by a job with lo == hi == UINT64_MAX */
  for (oracle_range_job *j = jobs; !(j->lo == UINT64_MAX && j->hi == UINT64_MAX); ++j)
    oracle_scan_range(j);
  return NULL;
}

static int oracle_pow(uint32_t D, uint32_t Q, uint64_t *out) {
  uint64_t n = 1;
  for (uint32_t q = 0; q < Q; ++q) {
    if (n > (1ULL << 48) / D) return ORACLE_E_RANGE;
    n *= D;
  }
  if (n > (1ULL << 48)) return ORACLE_E_RANGE;
  *out = n;
  return ORACLE_OK;
}

/*
 * oracle_map: brute-force argmin for `epochs` independent epochs.
 *   K, X        [epochs][Q][D] uint64, host memory, C order
 *   lo, hi      index range searched in every epoch; hi == 0 means the full range [0, D^Q)
 *   threads     worker threads (>= 1)
 *   index_out   [epochs] lowest index of a minimum-makespan mapping in [lo, hi)
 *   makespan_out[epochs] its makespan
 *   mapping_out [epochs][Q] its device tuple, or NULL
 * Returns ORACLE_OK, ORACLE_E_INVAL (Q, D, pointers, range) or ORACLE_E_RANGE.
 *
 * oracle_map_constrained additionally takes
 *   base        [epochs][D] loads already on each device (queues pinned outside the pool:
 *               SCHED_OFF queues), or NULL for all zero;
 *   elig        [epochs][Q] bit masks of the devices each queue may use (bit d = device
 *               d; 0 = any device), or NULL. Mappings outside the masks are not candidates.
 * An epoch whose range holds no feasible mapping yields ORACLE_E_INVAL.
 */
int oracle_map_constrained(uint32_t Q, uint32_t D, uint64_t epochs, const uint64_t *K,
                           const uint64_t *X, const uint64_t *base, const uint16_t *elig,
                           uint64_t lo, uint64_t hi, int threads, uint64_t *index_out,
                           uint64_t *makespan_out, uint8_t *mapping_out) {
  if (Q == 0 || D == 0 || Q > ORACLE_MAX_Q || D > ORACLE_MAX_D) return ORACLE_E_INVAL;
  if (epochs == 0) return ORACLE_OK;
  if (!K || !X || !index_out || !makespan_out) return ORACLE_E_INVAL;
  uint64_t N;
  if (oracle_pow(D, Q, &N) != ORACLE_OK) return ORACLE_E_RANGE;
  if (hi == 0) hi = N;
  if (lo >= hi || hi > N) return ORACLE_E_INVAL;
  for (uint64_t i = 0; i < epochs * Q * D; ++i)
    if (K[i] >= ORACLE_ENTRY_LIMIT || X[i] >= ORACLE_ENTRY_LIMIT) return ORACLE_E_RANGE;
  if (base)
    for (uint64_t i = 0; i < epochs * D; ++i)
      if (base[i] >= ORACLE_ENTRY_LIMIT) return ORACLE_E_RANGE;
  if (threads < 1) threads = 1;

  /* work split: whole epochs per thread when there are enough epochs, otherwise every
     epoch's range is cut into `threads` contiguous pieces */
  uint64_t pieces = (epochs >= (uint64_t)threads) ? 1 : (uint64_t)threads;
  if (pieces > hi - lo) pieces = hi - lo;
  uint64_t njobs = epochs * pieces;
  oracle_range_job *jobs = (oracle_range_job *)calloc(njobs, sizeof(oracle_range_job));
  if (!jobs) return ORACLE_E_INVAL;
  for (uint64_t e = 0; e < epochs; ++e)
    for (uint64_t p = 0; p < pieces; ++p) {
      oracle_range_job *j = &jobs[e * pieces + p];
      j->Q = Q;
      j->D = D;
      j->K = K + e * Q * D;
      j->X = X + e * Q * D;
      j->base = base ? base + e * D : NULL;
      j->elig = elig ? elig + e * Q : NULL;
      j->lo = lo + (hi - lo) * p / pieces;
      j->hi = lo + (hi - lo) * (p + 1) / pieces;
    }
  /* distribute jobs to threads contiguously, each list terminated by a sentinel */
  int nt = threads;
  if ((uint64_t)nt > njobs) nt = (int)njobs;
  oracle_range_job **lists = (oracle_range_job **)calloc((size_t)nt, sizeof(*lists));
  pthread_t *tid = (pthread_t *)calloc((size_t)nt, sizeof(pthread_t));
  for (int t = 0; t < nt; ++t) {
    uint64_t a = njobs * (uint64_t)t / (uint64_t)nt, b = njobs * (uint64_t)(t + 1) / (uint64_t)nt;
    lists[t] = (oracle_range_job *)calloc(b - a + 1, sizeof(oracle_range_job));
    memcpy(lists[t], jobs + a, (b - a) * sizeof(oracle_range_job));
    lists[t][b - a].lo = UINT64_MAX;
    lists[t][b - a].hi = UINT64_MAX;
  }
  for (int t = 1; t < nt; ++t) pthread_create(&tid[t], NULL, oracle_thread_main, lists[t]);
  oracle_thread_main(lists[0]);
  for (int t = 1; t < nt; ++t) pthread_join(tid[t], NULL);
  for (int t = 0; t < nt; ++t) {
    uint64_t a = njobs * (uint64_t)t / (uint64_t)nt, b = njobs * (uint64_t)(t + 1) / (uint64_t)nt;
    memcpy(jobs + a, lists[t], (b - a) * sizeof(oracle_range_job));
    free(lists[t]);
  }
  free(lists);
  free(tid);

  /* merge pieces of each epoch lexicographically by (makespan, index) */
  for (uint64_t e = 0; e < epochs; ++e) {
    uint64_t bms = 0, bm = 0;
    int have = 0;
    for (uint64_t p = 0; p < pieces; ++p) {
      oracle_range_job *j = &jobs[e * pieces + p];
      if (!j->found) continue;
      if (!have || j->best_ms < bms || (j->best_ms == bms && j->best_m < bm)) {
        bms = j->best_ms;
        bm = j->best_m;
        have = 1;
      }
    }
    index_out[e] = bm;
    makespan_out[e] = bms;
    if (mapping_out) {
      uint64_t rest = bm;
      for (int q = (int)Q - 1; q >= 0; --q) {
        mapping_out[e * Q + (uint64_t)q] = (uint8_t)(rest % D);
        rest /= D;
      }
    }
    if (!have) {  /* no feasible mapping in the range */
      free(jobs);
      return ORACLE_E_INVAL;
    }
  }
  free(jobs);
  return ORACLE_OK;
}

/* The unconstrained mapper: no pre-existing loads, every device eligible. */
int oracle_map(uint32_t Q, uint32_t D, uint64_t epochs, const uint64_t *K, const uint64_t *X,
               uint64_t lo, uint64_t hi, int threads, uint64_t *index_out, uint64_t *makespan_out,
               uint8_t *mapping_out) {
  return oracle_map_constrained(Q, D, epochs, K, X, NULL, NULL, lo, hi, threads, index_out,
                                makespan_out, mapping_out);
}

/* oracle_score: makespan of one given mapping (digit tuple). Used by
   tests to re-score a returned mapping and by the Fig. 4 schedule upper bounds. */
uint64_t oracle_score(uint32_t Q, uint32_t D, const uint64_t *K, const uint64_t *X,
                      const uint8_t *mapping) {
  uint64_t load[ORACLE_MAX_D];
  for (uint32_t d = 0; d < D; ++d) load[d] = 0;
  for (uint32_t q = 0; q < Q; ++q) load[mapping[q]] += K[q * D + mapping[q]] + X[q * D + mapping[q]];
  uint64_t ms = 0;
  for (uint32_t d = 0; d < D; ++d)
    if (load[d] > ms) ms = load[d];
  return ms;
}

/* oracle_score_base: makespan of one mapping on devices that already carry `base` loads
   ([D], or NULL for zero) -- the same definition with SCHED_OFF queues' loads included. */
uint64_t oracle_score_base(uint32_t Q, uint32_t D, const uint64_t *K, const uint64_t *X,
                           const uint64_t *base, const uint8_t *mapping) {
  uint64_t load[ORACLE_MAX_D];
  for (uint32_t d = 0; d < D; ++d) load[d] = base ? base[d] : 0;
  for (uint32_t q = 0; q < Q; ++q) load[mapping[q]] += K[q * D + mapping[q]] + X[q * D + mapping[q]];
  uint64_t ms = 0;
  for (uint32_t d = 0; d < D; ++d)
    if (load[d] > ms) ms = load[d];
  return ms;
}
