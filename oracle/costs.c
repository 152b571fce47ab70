/*
 * oracle/costs.c -- TEST INFRASTRUCTURE ONLY (see oracle.c's header; same rules: the
 * product never calls this, this includes nothing from the product).
 *
 * Cost-table construction, the step that feeds the mapper its per-queue
 * aggregate costs, written out plainly from the paper's description:
 *
 *  * kernel part (PAPER.md L1008-1040 kernel profiler: "we run the kernels once per device
 *    and store the corresponding execution times as part of the kernel profile";
 *    L1134-1164: a kernel epoch's value is "the aggregate performance vector of the epoch on
 *    all the devices"):   K[e][q][d] = sum over the kernel invocations enqueued to queue q in
 *    epoch e of profile[kernel][d]        (reading R15: invocations are a multiset, summed)
 *
 *  * transfer part (PAPER.md L877-913 device profiler: H2D bandwidths per device measured
 *    over data sizes "from being latency bound to bandwidth bound", "bandwidth numbers for
 *    unknown data sizes are computed by using simple interpolation"; L1293-1301: a transfer
 *    between devices is "a D2H-H2D double operation via the host memory"; L1309-1321: data
 *    cached on a device needs no transfer):
 *      X[e][q][d] = 0                                   if the data is on d or cached on d
 *                 = t_h2d(d, bytes)                     if the data is in host memory
 *                 = t_d2h(src, bytes) + t_h2d(d, bytes) if it is on another device src
 *    where a device flagged host_shared (an OpenCL CPU device working on host memory) has
 *    t_h2d = t_d2h = 0, and
 *      t(curve, bytes) = ceil(bytes / bw(bytes)) ns, bw linearly interpolated in bytes
 *      between the two neighbouring sample sizes, clamped to the first / last sample
 *    (reading R16). All arithmetic in IEEE fp64, no fused multiply-add (-ffp-contract=off),
 *    in exactly the order written below.
 *
 *  * sockets ("Benchmarks measuring host-to-device (H2D) bandwidths are
 *    run for all the CPU socket-device combinations"; L1349-1361: "nonuniform host-device
 *    ... distances ... depending on the core affinity of the host thread"; reading R19): the
 *    curves are per (socket, device), and queue q's host memory -- its data when
 *    source = -1, the staging buffer of a D2H-H2D double operation otherwise -- is on socket
 *    host_socket[e][q]; both legs use that socket's curves. One socket = the plain model.
 *
 *  * range (reading R10): a profile entry >= 2^48, or a running kernel sum that
 *    reaches 2^48, is COST_E_RANGE (the sum is checked after every addition, so it never
 *    wraps), as is any finished cost >= 2^48.
 */
#include <math.h>
#include <stdint.h>

#define COST_OK 0
#define COST_E_INVAL (-1)
#define COST_E_RANGE (-2)

/* bandwidth (bytes/ns) of one curve at `bytes`: linear interpolation between samples */
static double oracle_bandwidth(uint32_t M, const uint64_t *sizes, const double *bw, uint64_t bytes) {
  if (bytes <= sizes[0]) return bw[0];
  if (bytes >= sizes[M - 1]) return bw[M - 1];
  uint32_t i = 0;
  while (!(sizes[i] <= bytes && bytes < sizes[i + 1])) ++i;
  double f = (double)(bytes - sizes[i]) / (double)(sizes[i + 1] - sizes[i]);
  return bw[i] + f * (bw[i + 1] - bw[i]);
}

/* integer ns to move `bytes` over one curve */
static uint64_t oracle_transfer_ns(uint32_t M, const uint64_t *sizes, const double *bw, uint64_t bytes) {
  if (bytes == 0) return 0;
  double t = (double)bytes / oracle_bandwidth(M, sizes, bw, bytes);
  return (uint64_t)ceil(t);
}

/*
 * oracle_build_costs: K and X for E epochs of Q queues on D devices.
 *   profile   [num_kernels][D] ns per invocation (each < 2^48)
 *   offsets   [E*Q + 1] CSR offsets of (e, q) into kernel_ids
 *   kernel_ids[offsets[E*Q]] kernel ids
 *   bytes     [E][Q] working-set size of each queue
 *   source    [E][Q] device holding the data, -1 = host memory
 *   cached    [E][Q] bit d: a copy is already on device d, or NULL
 *   sizes     [M] ascending sample sizes
 *   num_sockets S >= 1 host sockets; h2d_bw, d2h_bw [S][D][M] bytes/ns (> 0)
 *   host_socket [E][Q] socket of the queue's host memory (< S), or NULL = socket 0
 *   host_shared bit d: device d works on host memory
 * Returns COST_OK, COST_E_INVAL (bad id / source / socket / offsets / curve) or COST_E_RANGE
 * (a profile entry, running sum or cost >= 2^48).
 */
int oracle_build_costs(uint32_t Q, uint32_t D, uint64_t E, uint32_t num_kernels,
                       const uint64_t *profile, const uint64_t *offsets,
                       const uint32_t *kernel_ids, const uint64_t *bytes, const int32_t *source,
                       const uint16_t *cached, uint32_t M, const uint64_t *sizes,
                       uint32_t num_sockets, const uint8_t *host_socket,
                       const double *h2d_bw, const double *d2h_bw, uint32_t host_shared,
                       uint64_t *K, uint64_t *X) {
  if (Q == 0 || D == 0 || D > 16 || M == 0 || num_sockets == 0) return COST_E_INVAL;
  for (uint32_t i = 0; i + 1 < M; ++i)
    if (!(sizes[i] < sizes[i + 1])) return COST_E_INVAL;
  for (uint64_t i = 0; i < (uint64_t)num_sockets * D * M; ++i)
    if (!(h2d_bw[i] > 0.0) || !(d2h_bw[i] > 0.0)) return COST_E_INVAL;
  for (uint64_t i = 0; i < (uint64_t)num_kernels * D; ++i)
    if (profile[i] >= (1ULL << 48)) return COST_E_RANGE;
  for (uint64_t e = 0; e < E; ++e)
    for (uint32_t q = 0; q < Q; ++q) {
      uint64_t eq = e * Q + q;
      if (offsets[eq + 1] < offsets[eq]) return COST_E_INVAL;
      /* kernel part: sum of the invoked kernels' profiled times on each device */
      for (uint32_t d = 0; d < D; ++d) {
        uint64_t sum = 0;
        for (uint64_t j = offsets[eq]; j < offsets[eq + 1]; ++j) {
          if (kernel_ids[j] >= num_kernels) return COST_E_INVAL;
          sum += profile[(uint64_t)kernel_ids[j] * D + d];
          if (sum >= (1ULL << 48)) return COST_E_RANGE;
        }
        K[eq * D + d] = sum;
      }
      /* transfer part: the queue's host memory is on socket s; both legs use s's curves */
      int32_t src = source[eq];
      if (src < -1 || src >= (int32_t)D) return COST_E_INVAL;
      uint32_t s = host_socket ? host_socket[eq] : 0;
      if (s >= num_sockets) return COST_E_INVAL;
      const double *h2d_s = h2d_bw + (uint64_t)s * D * M;
      const double *d2h_s = d2h_bw + (uint64_t)s * D * M;
      for (uint32_t d = 0; d < D; ++d) {
        uint64_t x;
        int on_d = (src == (int32_t)d) || (cached && ((cached[eq] >> d) & 1u));
        if (on_d) {
          x = 0;
        } else {
          uint64_t up = 0, down = 0;
          if (!((host_shared >> d) & 1u)) up = oracle_transfer_ns(M, sizes, h2d_s + (uint64_t)d * M, bytes[eq]);
          if (src >= 0 && !((host_shared >> (uint32_t)src) & 1u))
            down = oracle_transfer_ns(M, sizes, d2h_s + (uint64_t)src * M, bytes[eq]);
          x = down + up;
        }
        X[eq * D + d] = x;
      }
      for (uint32_t d = 0; d < D; ++d)
        if (K[eq * D + d] >= (1ULL << 48) || X[eq * D + d] >= (1ULL << 48)) return COST_E_RANGE;
    }
  return COST_OK;
}
