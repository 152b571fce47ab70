/*
 * mcl_ext.h -- measurement and communicator helpers of libmcl.so (C ABI).
 *
 * Not needed to use the mapper (that is include/mcl.h); used by bench.py and the tests to
 * time the search kernel on its own stream, to measure the integer-pipe peak that bounds it
 * (SURVEY.md SS8(d) roofline, component N7), and to build an NCCL communicator without a
 * torch process group.
 */
#ifndef MCL_EXT_H_
#define MCL_EXT_H_

#include <stdint.h>

#include "mcl.h"

#ifdef __cplusplus
extern "C" {
#endif

/* Enable (1) / disable (0) CUDA-event timing of the main search kernel of every
   mcl_map_queues call on h. Events are recorded on the stream the kernel is launched on. */
mcl_status_t mcl_set_timing(mcl_mapper_t* h, int enable);

/* Device time in milliseconds of the main search kernel of the last call (timing >= 1),
   and of the whole device-side sequence of that call, staging copies included (timing 2;
   else 0). enable: 0 = off, 1 = search kernel only (two events), 2 = kernel and call. */
mcl_status_t mcl_last_kernel_time(const mcl_mapper_t* h, float* kernel_ms, float* call_ms);

/* Measurement aid for the timing events (not part of any step): with hold_us > 0, every
   timed launch is preceded on the same stream by a one-thread kernel that spins for
   hold_us microseconds (%globaltimer), so the host-side launch latency elapses while the
   stream is busy and the kernel_ms events bracket the search kernel's device execution
   only. 0 (default) disables it. Has no effect unless timing is enabled. */
mcl_status_t mcl_set_timing_hold(mcl_mapper_t* h, uint32_t hold_us);

/*
 * Integer-pipe throughput probe on `device` (op: 0 = 2-input min/max VIMNMX, 1 = 3-input
 * VIMNMX3, 2 = IADD3, 3 = IMAD, 4 = VIMNMX3 and IMAD interleaved). Runs for ~1 ms at full
 * occupancy and reports lane-operations per second, lane-operations per SM clock, and the
 * effective SM clock in MHz over the run. Synchronous. Any output pointer may be NULL.
 */
mcl_status_t mcl_probe_int_rate(int device, int op, double* lane_ops_per_s,
                                double* lane_ops_per_clk_sm, double* eff_mhz);

/*
 * Launch floor on `device`: the mean over `reps` (>= 1) of what CUDA events report around
 * a kernel that does nothing (one CTA of 512 threads per SM), each timed as the search
 * kernels are timed by mcl_set_timing + mcl_set_timing_hold(200), and of the events alone.
 * It is the part of every event-timed kernel duration that no kernel can avoid on this
 * platform. Synchronous, on the legacy default stream. Any output pointer may be NULL.
 * MCL_E_INVAL for a bad device or reps < 1.
 */
mcl_status_t mcl_probe_launch_floor(int device, int reps, double* empty_kernel_us, double* events_only_us);

/* Testing aid: force the kernel of later mcl_map_queues calls on h. path: 0 = automatic
   (default), 1 = register-blocked (u32 loads, falls back to 64-bit when a bound needs it),
   2 = register-blocked with 64-bit loads, 3 = generic, 4 = small batched, 5 = register-
   blocked u32 over a flattened (epoch, block) space (batched calls), 6 = always run the
   branch-and-bound kernel in mcl_map_queues_pruned (no small-space cutover), 7 = warp-per-
   epoch batched kernel (unconstrained single-GPU batches of the shapes it is instantiated
   for; chosen automatically from one full wave of epochs), 8 = mixed-radix constrained
   kernel (calls with eligible-device masks, 2 <= D <= 8, Q >= 3; the automatic choice for
   them -- force 1 for the INF-masked full-space blocked kernel instead), 9 = its warp-per-
   epoch form for batches (single GPU, at most 2^16 reduced blocks per epoch; chosen
   automatically from four epochs per SM). A path that does not support (Q, D) or the
   handle's sharding makes the call fail with MCL_E_INVAL. */
mcl_status_t mcl_force_path(mcl_mapper_t* h, int path);

/* Pipelined staging of host-resident batches. When every cost table and output of an
   unconstrained single-GPU mcl_map_queues call is host memory, the epochs are cut into
   chunks whose host->device copies, search and device->host copies are issued on three
   rotating streams, so the PCIe copies of one chunk overlap the search of another (the copy
   engines run both directions at once). Results are identical to the unpipelined call
   (epochs are independent). chunks: 0 = automatic (default: at least 1.5 MB of K + X per
   chunk, at most 4 chunks, each at least one wave of the warp-per-epoch kernel: 16 epochs
   per SM), 1 = off, n > 1 = exactly min(n, epochs) chunks. With three or more chunks the
   first and the last hold half as many epochs as the others (a short first copy before the
   first search, a short search after the last copy). mcl_last_launch_info's info[7] is the
   number of chunks of a pipelined call (0 otherwise). Calls whose buffers are pinned host
   memory skip staging altogether when they are small (MCL_ZERO_COPY_MAX bytes, default
   64 KiB) or run the warp-per-epoch batch kernel (which reads each epoch's costs one epoch
   ahead, so PCIe reads overlap the search): the kernels use them in place, zero-copy --
   unless n > 1 forces the pipeline.
   Errors: MCL_E_INVAL (NULL h, n < 0). */
mcl_status_t mcl_set_pipeline_chunks(mcl_mapper_t* h, int chunks);

/* Number of SMs of `device` (for roofline bookkeeping). */
mcl_status_t mcl_device_sms(int device, int* sms);

/* NCCL communicator helpers (libnccl.so.2 is resolved at run time, reusing the copy
   torch already loaded when there is one). The unique id is 128 opaque bytes that rank 0
   creates and every rank passes to mcl_comm_init; the communicator belongs to the caller
   and is released with mcl_comm_destroy. */
mcl_status_t mcl_comm_unique_id(uint8_t id_out[128]);
mcl_status_t mcl_comm_init(int device, int world, int rank, const uint8_t id[128], void** comm_out);
mcl_status_t mcl_comm_destroy(void* comm);

#ifdef __cplusplus
}
#endif

#endif /* MCL_EXT_H_ */
