/*
 * mcl.h -- C ABI of the B200-native MultiCL device-mapper search (libmcl.so).
 *
 * The operation (Aji, Pena, Balaji, Feng, IEEE CLUSTER 2015, SS V.A
 * "Device Mapper": "apply a simple dynamic programming approach to determine the ideal
 * queue-device mapping that minimizes the concurrent execution time"; PAPER.md
 * L2106-2118, SS VI.B.1: the scheduler "computes the aggregate cost metric from the data
 * transfer and kernel execution costs"), per scheduling epoch e:
 *
 *   C[q][d]   = cost_kernel[e][q][d] + cost_xfer[e][q][d]        (integer ns)
 *   m         = sum_q d_q * D^(Q-1-q)     mapping index, queue 0 most significant digit
 *   L_d(m)    = sum over queues q placed on device d of C[q][d]   (queues on one device
 *               serialise; an idle device has load 0)
 *   ms(m)     = max_d L_d(m)              (distinct devices run concurrently)
 *   result    = the LOWEST index m* among the mappings with minimal ms, its digits and ms.
 *
 * All D^Q mappings are scored exhaustively on the GPU (hand-written sm_100a kernels).
 * Costs are exact unsigned integers, so results are bit-exact (no tolerance).
 *
 * Threading: a handle is used by one host thread at a time. Different handles are
 * independent. All calls are synchronous: they return after every output is written.
 */
#ifndef MCL_H_
#define MCL_H_

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct mcl_mapper mcl_mapper_t; /* opaque; owned by the library */

typedef enum {
  MCL_OK = 0,
  MCL_E_INVAL = -1,  /* NULL required pointer, Q == 0, D == 0, D > 16, Q > 32, bad config */
  MCL_E_RANGE = -2,  /* D^Q > 2^48, or some cost entry >= 2^48 */
  MCL_E_CUDA = -3,   /* a CUDA runtime call failed (see mcl_last_error_string) */
  MCL_E_NCCL = -4,   /* an NCCL call failed, or NCCL could not be loaded */
  MCL_E_NOMEM = -5   /* device / pinned-host allocation failed */
} mcl_status_t;

#define MCL_MAX_QUEUES 32
#define MCL_MAX_DEVICES 16
#define MCL_MAX_ENTRY_BITS 48 /* every cost entry must be < 2^48 */
#define MCL_MAX_INDEX_BITS 48 /* D^Q must be <= 2^48 */

typedef struct {
  int device;      /* CUDA device ordinal this handle runs on                            */
  void* stream;    /* cudaStream_t to run on (cudaStreamLegacy = (void*)1 and cudaStreamPerThread
                      = (void*)2 are accepted); NULL = a non-blocking stream owned by the handle,
                      which is not ordered after work on any other stream                  */
  void* nccl_comm; /* ncclComm_t (e.g. torch ProcessGroupNCCL._comm_ptr()) or NULL        */
  int rank;        /* this process's shard, 0 <= rank < world                             */
  int world;       /* number of shards; 0 or 1 = the whole index space                    */
} mcl_config_t;

/*
 * Create a mapper handle on cfg->device.
 *   cfg  : required. With nccl_comm == NULL and world > 1 the handle searches only shard
 *          `rank` of every epoch's index space and returns that shard's local argmin (a
 *          sub-range search; used to test sharding on one GPU). With nccl_comm != NULL,
 *          rank/world must equal the communicator's and every mcl_map_queues call is
 *          COLLECTIVE (see below).
 *   out  : receives the handle. The handle owns its scratch (per-CTA partial results,
 *          staging buffers, a mapped host status word), allocated here and grown on demand.
 * Errors: MCL_E_INVAL (NULL pointers, bad rank/world, bad device), MCL_E_CUDA, MCL_E_NOMEM,
 *         MCL_E_NCCL (nccl_comm given but libnccl could not be resolved).
 */
mcl_status_t mcl_mapper_create(const mcl_config_t* cfg, mcl_mapper_t** out);

/*
 * Find the minimum-makespan queue->device mapping of every epoch.
 *   Q, D          : queues and devices; 1 <= Q <= 32, 1 <= D <= 16, D^Q <= 2^48.
 *   epochs        : number of independent epochs E (0 = no-op, returns MCL_OK).
 *   cost_kernel   : [E][Q][D] uint64, C order: per-queue aggregate kernel time on each
 *                   device (the kernel profiler's output).
 *   cost_xfer     : [E][Q][D] uint64, C order: cost of moving the queue's buffers to each
 *                   device (derived from the device profiles).
 *   mapping_index : [E] uint64 out: lowest index of an optimal mapping.
 *   mapping       : [E][Q] uint8 out: its device per queue (digit q of the index), or NULL.
 *   makespan      : [E] uint64 out: its makespan, in the same unit as the costs.
 * Every pointer may be device memory (the fast path: no copies) or host memory (pageable
 * or pinned; detected with cudaPointerGetAttributes and staged through handle-owned device
 * buffers inside the call; a small call whose buffers are pinned host memory uses them in
 * place, zero-copy over PCIe). A pointer the CUDA runtime cannot classify is MCL_E_INVAL;
 * pageable host pointers cannot be validated and are trusted, as with any C library taking
 * host buffers. The caller owns all buffers; the library never frees them.
 * Inputs are only read; outputs are fully written on MCL_OK and unspecified on error.
 * Stream order: device inputs must be complete, and device outputs free to overwrite, in
 * the order of the handle's stream (cfg->stream). Pass the stream that produced the inputs
 * (cudaStreamLegacy = (void*)1 for the legacy default stream); with cfg->stream == NULL the
 * handle's own non-blocking stream does NOT wait for work on other streams.
 *
 * Sharding: the index space [0, D^Q) of each epoch is cut into `world` contiguous ranges
 * [floor(r*N/G), floor((r+1)*N/G)) (in whole blocks of the innermost digits). With a
 * communicator, each rank searches its range and one ncclAllReduce(MIN, uint64) over the
 * packed key (makespan << index_bits | index) combines them, so every rank receives the
 * identical global result (bit-identical for every world size). When the makespan does not
 * fit beside the index in 64 bits, a two-step reduction (min makespan, then min index
 * among the ranks holding it) is used instead. All ranks must pass identical inputs.
 *
 * Errors: MCL_E_INVAL (NULL required pointer, Q/D out of bounds), MCL_E_RANGE (D^Q > 2^48
 *         or an entry >= 2^48, detected on the device), MCL_E_CUDA, MCL_E_NCCL.
 */
mcl_status_t mcl_map_queues(mcl_mapper_t* h, uint32_t Q, uint32_t D, uint64_t epochs,
                            const uint64_t* cost_kernel, const uint64_t* cost_xfer,
                            uint64_t* mapping_index, uint8_t* mapping, uint64_t* makespan);

/*
 * Fused cross-GPU exchange (no paper counterpart -- the paper's mapper is
 * single-host). Replaces the NCCL all-reduce of a sharded handle by an
 * exchange INSIDE the search kernel over NVLink / NVSwitch peer memory: each rank owns an
 * exchange slab in its device memory, exported as a CUDA IPC handle and mapped by every
 * other rank. When the rank's search is done, the kernel's last CTA adds its packed keys to
 * every rank's slab with system-scope atomicMin, signals every rank, waits for all `world`
 * signals and decodes the global result: one launch per call, no collective library, no
 * extra kernel. The result is the same as the NCCL path's (including the two-step
 * lexicographic reduction when a makespan does not fit beside the index).
 * Setup, collective over the handle's `world` ranks (cfg->rank / cfg->world), once:
 *   1. every rank: mcl_peer_export(h, max_epochs, handle_out) -> 64 opaque bytes
 *      (allocates the slab: 2 * max_epochs + 8 words, max_epochs in [1, 2^20]);
 *   2. the ranks exchange the bytes out of band (e.g. torch.distributed all_gather);
 *   3. every rank: mcl_peer_import(h, handles, timeout_ms), handles = [world][64] bytes
 *      in rank order (a rank's own entry is not opened; world == 1 exchanges with itself).
 * Afterwards every mcl_map_queues / mcl_map_queues_constrained call on h with
 * epochs <= max_epochs is COLLECTIVE through the slabs: all ranks must make the same calls,
 * in the same order, with identical inputs. A communicator, if the handle has one, still
 * serves larger calls; without one (world > 1), a larger call fails with MCL_E_INVAL
 * instead of returning a shard-local result. If some rank does not signal within
 * timeout_ms (0 = 30 s), the call fails with MCL_E_NCCL ("peer exchange timed out")
 * instead of hanging, and the handle's exchange is disabled: later calls go to the
 * communicator, or (without one) fail with MCL_E_NCCL until a new export / import. Destroy the handles of all ranks together (a rank's slab stays
 * mapped by its peers until they destroy theirs).
 * Errors: MCL_E_INVAL (bad arguments, world handles not matching, import before export),
 *         MCL_E_CUDA (IPC export/open failed, e.g. no peer access between the devices).
 */
mcl_status_t mcl_peer_export(mcl_mapper_t* h, uint64_t max_epochs, uint8_t handle_out[64]);
mcl_status_t mcl_peer_import(mcl_mapper_t* h, const uint8_t* handles, uint32_t timeout_ms);

/*
 * Constrained variant. The paper's runtime maps only the SCHED_AUTO queues
 * of the pool; queues created with SCHED_OFF "will be statically mapped to the chosen
 * device" and still occupy it. Here:
 *   base_load : [E][D] uint64 or NULL -- load already on each device (e.g. the SCHED_OFF
 *               queues' cost); every device's load starts from it. Entries < 2^48.
 *   eligible  : [E][Q] uint16 or NULL -- bit d set = queue q may run on device d; 0 = any
 *               device. A queue pinned to one device has a single bit.
 * The result is the lowest index (in the full D^Q index space) among the mappings that
 * respect every mask and minimise max_d (base_load[d] + sum of C over the queues on d).
 * Either pointer may be NULL; both NULL is mcl_map_queues. Same buffer rules and errors as
 * mcl_map_queues, plus MCL_E_INVAL when some queue has no eligible device < D.
 * With masks (2 <= D <= 8, Q >= 3) only the FEASIBLE mappings are enumerated (a true
 * mixed-radix search): a pinned queue (one eligible device) leaves the enumeration -- its
 * cost joins its device's base load, its digit is a constant of the index -- and the other
 * queues run over their eligible devices only (the last three queues over all D devices with
 * ineligible entries excluded), so the work is proportional to the product of the queues'
 * eligible-device counts, not to D^Q. Sharding then cuts this feasible enumeration (in
 * increasing full-index order) into `world` contiguous ranges, per epoch; without masks it
 * cuts the full index space as in mcl_map_queues. A shard-mode handle (world > 1, no
 * communicator) whose range holds no feasible mapping reports index = makespan = UINT64_MAX
 * and mapping bytes 0xFF for that epoch.
 */
typedef struct {
  const uint64_t* base_load; /* [E][D] or NULL */
  const uint16_t* eligible;  /* [E][Q] or NULL */
} mcl_constraints_t;

mcl_status_t mcl_map_queues_constrained(mcl_mapper_t* h, uint32_t Q, uint32_t D, uint64_t epochs,
                                        const uint64_t* cost_kernel, const uint64_t* cost_xfer,
                                        const mcl_constraints_t* constraints,
                                        uint64_t* mapping_index, uint8_t* mapping,
                                        uint64_t* makespan);

/*
 * Exact search with pruning: returns exactly what
 * mcl_map_queues_constrained returns (the lowest-index minimum-makespan mapping), found by
 * a parallel depth-first branch and bound over the queue digits (lower bounds: the current
 * max load, the largest remaining per-queue minimum cost, and the total work spread over D
 * devices) instead of scoring all D^Q mappings. Its cost depends on the instance
 * (time-to-solution, not mappings/s); random instances of 10^10-10^14 mappings typically
 * need 10^2-10^6 nodes. Ineligible devices are skipped outright (a true mixed-radix
 * search). The handle's sharding is ignored: every call solves the whole index space (a
 * collective handle gets the same answer on every rank without communication).
 * constraints may be NULL. mcl_last_launch_info's info[0] = 6 and info[7] = nodes visited.
 * Same buffer rules and errors as mcl_map_queues_constrained.
 */
mcl_status_t mcl_map_queues_pruned(mcl_mapper_t* h, uint32_t Q, uint32_t D, uint64_t epochs,
                                   const uint64_t* cost_kernel, const uint64_t* cost_xfer,
                                   const mcl_constraints_t* constraints, uint64_t* mapping_index,
                                   uint8_t* mapping, uint64_t* makespan);

/*
 * Cost-table construction: the mapper's inputs built on the GPU from the
 * runtime's profiles.
 *   K[e][q][d] = sum over the kernel invocations enqueued to queue q in epoch e of
 *                kernel_profile[kernel][d]  (kernel profiler: each kernel run once per
 *                device; an epoch's "aggregate performance vector",
 *                L1154-1158). Repeated invocations count each time.
 *   X[e][q][d] = 0 if the queue's data is on device d (source == d) or a copy is cached
 *                there (cached bit d, L1309-1321); else t_h2d(d) when the data is in host
 *                memory (source == -1), or t_d2h(source) + t_h2d(d) when it is on another
 *                device ("a D2H-H2D double operation via the host memory", L1293-1301). A
 *                device with host_shared bit d set (an OpenCL CPU device on host memory)
 *                has no H2D / D2H leg. t(curve, bytes) = ceil(bytes / bw(bytes)) ns with bw
 *                (bytes per ns) linearly interpolated in bytes between the two neighbouring
 *                sampled sizes and clamped outside them (device profiler: bandwidths over
 *                sizes "from latency bound to bandwidth bound", "simple interpolation
 *                techniques" for other sizes, L877-913); IEEE fp64, no fused multiply-add.
 *                The curves are per host socket ("H2D bandwidths are run for all the CPU
 *                socket-device combinations", L897-901; nonuniform host-device distances,
 *                L1349-1361): queue q's host memory -- its data, or the staging buffer of a
 *                D2H-H2D double operation -- is on socket host_socket[e][q], and both legs
 *                use that socket's curves.
 * Every array may be host or device memory (host arrays are staged). K sums are exact: a
 * profile entry >= 2^48 or a sum reaching 2^48 is MCL_E_RANGE (never a wrapped value).
 */
typedef struct {
  uint32_t num_kernels;            /* rows of kernel_profile                             */
  const uint64_t* kernel_profile;  /* [num_kernels][D] ns per invocation on each device  */
  const uint64_t* offsets;         /* [E*Q + 1] CSR offsets of (e, q) into kernel_ids     */
  const uint32_t* kernel_ids;      /* [num_invocations] kernel of each invocation         */
  uint64_t num_invocations;        /* == offsets[E*Q]                                     */
  const uint64_t* bytes;           /* [E][Q] working-set bytes of each queue              */
  const int32_t* source;           /* [E][Q] device holding the data, -1 = host memory    */
  const uint16_t* cached;          /* [E][Q] devices already holding a copy, or NULL      */
  uint32_t num_sizes;              /* M sampled sizes, 1..64                              */
  const uint64_t* sizes;           /* [M] strictly ascending bytes                        */
  const double* h2d_bw;            /* [S][D][M] host->device bandwidth, bytes/ns, > 0     */
  const double* d2h_bw;            /* [S][D][M] device->host bandwidth, bytes/ns, > 0     */
  uint32_t host_shared;            /* bit d: device d works on host memory                */
  uint32_t num_sockets;            /* S host sockets, 1..8 (0 = 1)                        */
  const uint8_t* host_socket;      /* [E][Q] socket of each queue's host memory (< S), or
                                      NULL = socket 0                                      */
} mcl_cost_model_t;

/* Build K and X ([E][Q][D] uint64, host or device outputs). Errors: MCL_E_INVAL (NULL
   pointer, Q/D out of bounds, num_sizes outside 1..64, num_sockets above 8, a kernel id >=
   num_kernels, a source outside -1..D-1, a socket >= S, bad offsets, sizes not ascending or a
   bandwidth <= 0), MCL_E_RANGE (a profile entry, kernel sum or cost >= 2^48), MCL_E_CUDA. */
mcl_status_t mcl_build_costs(mcl_mapper_t* h, uint32_t Q, uint32_t D, uint64_t epochs,
                             const mcl_cost_model_t* model, uint64_t* cost_kernel,
                             uint64_t* cost_xfer);

/* The whole pipeline in one call: build K and X in handle-owned device memory, then run
   mcl_map_queues_constrained on them (constraints may be NULL). Outputs as mcl_map_queues. */
mcl_status_t mcl_map_from_profiles(mcl_mapper_t* h, uint32_t Q, uint32_t D, uint64_t epochs,
                                   const mcl_cost_model_t* model,
                                   const mcl_constraints_t* constraints,
                                   uint64_t* mapping_index, uint8_t* mapping, uint64_t* makespan);

/*
 * Score GIVEN mappings: makespan[e] = max_d (base_load[e][d] + sum over queues q with
 * mappings[e][q] == d of (cost_kernel + cost_xfer)[e][q][d]) -- e.g. a ROUND_ROBIN mapping
 * ("the next available device when the scheduler is triggered") or a
 * static hint-based choice (SS V.B), to compare a policy against the optimum.
 *   mappings : [E][Q] uint8 device ids (< D, else MCL_E_INVAL); base_load may be NULL.
 * Host or device pointers; synchronous; errors as mcl_map_queues.
 */
mcl_status_t mcl_score_mappings(mcl_mapper_t* h, uint32_t Q, uint32_t D, uint64_t epochs,
                                const uint64_t* cost_kernel, const uint64_t* cost_xfer,
                                const uint64_t* base_load, const uint8_t* mappings,
                                uint64_t* makespan);

/*
 * Static command-queue scheduling, the SCHED_AUTO_STATIC policy baseline (PAPER.md
 * L1088-1116, SS V.B: "we statically decide the command queue schedules based only on the
 * device profiles ... uses the command queue properties (compute intensive, memory
 * intensive, or I/O intensive) as the selection criterion and chooses the best available
 * device for the given command queue"; Table I's SCHED_COMPUTE_BOUND / SCHED_MEMORY_BOUND /
 * SCHED_IO_BOUND hints). No kernel profiles, no search: each queue independently.
 *   hints        : [E][Q] uint8 class of each queue, < num_classes (e.g. 0 = compute-bound,
 *                  1 = memory-bound, 2 = I/O-bound)
 *   num_classes  : 1..16
 *   device_score : [num_classes][D] uint64 device-profile cost of class c on device d (lower
 *                  is better, e.g. ns of the class's device benchmark)
 *   eligible     : [E][Q] uint16 or NULL -- as in mcl_map_queues_constrained ("available")
 *   mappings     : [E][Q] uint8 out: the eligible device with the lowest score for the
 *                  queue's class, ties to the lowest device id.
 * Score the result with mcl_score_mappings to compare the policy with the optimum.
 * Host or device pointers; synchronous. Errors: MCL_E_INVAL (NULL pointer, bad shape,
 * num_classes outside 1..16, a hint >= num_classes, a queue with no eligible device < D),
 * MCL_E_CUDA.
 */
mcl_status_t mcl_static_mappings(mcl_mapper_t* h, uint32_t Q, uint32_t D, uint64_t epochs,
                                 const uint8_t* hints, uint32_t num_classes,
                                 const uint64_t* device_score, const uint16_t* eligible,
                                 uint8_t* mappings);

/*
 * Resident mapper: low-latency online decisions (cfg1-sized searches). The paper's mapper
 * runs at every scheduling epoch on the application's critical path;
 * a launch per decision costs a launch, its ramp and a stream synchronisation (~15 us).
 * mcl_resident_start leaves ONE warp resident on the handle's device, polling a mailbox
 * in pinned, device-mapped host memory; mcl_resident_map writes the inputs and a request
 * number into it and spins until the warp publishes the answer (no launch, no copy engine,
 * no stream synchronisation per call). Same definition and outputs as mcl_map_queues.
 *   Q, D        : fixed per start; D^Q <= 8192 (the paper's largest decision: FT, 8 queues on
 *                 3 devices = 6561 mappings), Q <= 16, D <= 16.
 *   max_epochs  : epochs per mcl_resident_map call, 1..64.
 *   idle_ms     : the warp exits after this long without a request (0 = 100 ms); the next
 *                 mcl_resident_map relaunches it (one launch, then resident again).
 * mcl_resident_map: cost_kernel / cost_xfer [epochs][Q][D] and the outputs ([epochs],
 *   [epochs][Q] or NULL, [epochs]) are HOST pointers (pageable or pinned; copied through the
 *   mailbox); epochs <= max_epochs. Synchronous. One call at a time per handle.
 * While the warp is resident, device-wide synchronisation (cudaDeviceSynchronize,
 * torch.cuda.synchronize) waits for it to exit (at most idle_ms): call mcl_resident_stop
 * first. mcl_resident_stop (and mcl_mapper_destroy) stop the warp and free the mailbox.
 * Errors: MCL_E_INVAL (shape, epochs, device pointers, not started), MCL_E_RANGE (an entry
 * >= 2^48), MCL_E_NOMEM, MCL_E_CUDA (launch failure, or no answer within 2 s).
 */
mcl_status_t mcl_resident_start(mcl_mapper_t* h, uint32_t Q, uint32_t D, uint32_t max_epochs,
                                uint32_t idle_ms);
mcl_status_t mcl_resident_map(mcl_mapper_t* h, uint64_t epochs, const uint64_t* cost_kernel,
                              const uint64_t* cost_xfer, uint64_t* mapping_index,
                              uint8_t* mapping, uint64_t* makespan);
mcl_status_t mcl_resident_stop(mcl_mapper_t* h);

/* Destroy a handle (NULL-safe). Frees the handle's scratch; never the caller's buffers and
   never the NCCL communicator (its owner, e.g. the torch process group, keeps it). */
void mcl_mapper_destroy(mcl_mapper_t* h);

/* Static text for a status code. */
const char* mcl_status_string(mcl_status_t s);

/* Text of the last CUDA/NCCL error seen on this handle ("" if none). Valid until the next
   call on the handle. NULL handle: the last creation error of this thread. */
const char* mcl_last_error_string(const mcl_mapper_t* h);

/*
 * Introspection for tests and benchmarks (not needed to use the mapper).
 * mcl_last_launch_info fills, for the most recent successful mcl_map_queues call on h:
 *   info[0] = kernel path id (1 = register-blocked u32 search, 2 = register-blocked u64
 *             search, 3 = generic search, 4 = small batched (thread per epoch),
 *             5 = register-blocked u32 over a flattened (epoch, block) space,
 *             6 = branch and bound (mcl_map_queues_pruned), 7 = warp-per-epoch batched u32,
 *             8 = register-blocked u32, one-CTA-per-SM build (single epochs, D = 5),
 *             9 / 10 = mixed-radix constrained search over the feasible mappings, u32 / u64,
 *             11 = the same, one warp per epoch, for batches of constrained epochs,
 *             12 = batched u32 with one 16-warp CTA per SM sharing its epochs in parts)
 *   info[1] = number of kernels launched by the call, info[2] = CTAs of the main kernel,
 *   info[3] = threads per CTA, info[4] = 1 if an NCCL all-reduce ran, 2 if the fused peer
 *   exchange ran, info[5] = index bits of the packed key, info[6] = 1 if the two-step
 *   reduce ran, info[7] = nodes visited (mcl_map_queues_pruned) or the number of chunks of
 *   a pipelined host-resident call (mcl_set_pipeline_chunks in mcl_ext.h), else 0.
 */
mcl_status_t mcl_last_launch_info(const mcl_mapper_t* h, int64_t info[8]);

/* Library version string "mcl <major>.<minor> sm_100a". */
const char* mcl_version(void);

#ifdef __cplusplus
}
#endif

#endif /* MCL_H_ */
