/*
 * adapcc.h -- C ABI of the B200-native AdapCC hot path.
 *
 * What it computes: collective communication executed along an AdapCC
 * *strategy* -- M parallel sub-collectives, each a weighted spanning tree over
 * the ranks with its own data partition S_m and chunk size C_m (PAPER.md
 * §IV-D) -- under a ready-rank mask: only ready ranks contribute,
 * non-ready ranks act as relays and still receive the result (§IV-C,
 * P:L127-159).  Semantics are defined by the CPU oracle (oracle/, DESIGN.md
 * §3); the strategy text format is DESIGN.md §2.
 *
 * Conventions for every entry point:
 *   - Returns adapcc_result_t; 0 == ADAPCC_SUCCESS.  Never throws, never exits.
 *   - Pointers named *buf / *bufs are DEVICE pointers on the communicator's
 *     device, 16-byte aligned; otherwise ADAPCC_ERR_INVALID_ARGUMENT.
 *   - Synchronous errors (bad argument, bad strategy) are detected before
 *     anything is enqueued; they are deterministic given identical arguments,
 *     so all ranks fail together.
 *   - Device-side errors (watchdog timeout) are latched; read them with
 *     adapcc_get_async_error(), after which the communicator must be finalized.
 *   - Collective calls (allreduce/allgather/alltoall/set_strategy) must be
 *     issued in the same order with the same arguments (except buffers) on
 *     every rank; they are asynchronous and stream-ordered (the paper's Work
 *     Queue / Result Queue, become the CUDA stream).  Calls on one
 *     communicator must be ordered (one stream, or streams joined by events).
 *   - Ownership: the library owns its scratch arena, IPC mappings, plan tables
 *     and a host-mapped error word; the caller owns every buffer and stream.
 */
#ifndef ADAPCC_H
#define ADAPCC_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#if defined(__GNUC__)
#define ADAPCC_API __attribute__((visibility("default")))
#else
#define ADAPCC_API
#endif

#define ADAPCC_VERSION 1
#define ADAPCC_MAX_RANKS 64

typedef struct adapcc_comm_s* adapcc_comm_t;
typedef void* adapcc_stream_t; /* a cudaStream_t; NULL = legacy default stream */

typedef enum {
  ADAPCC_SUCCESS = 0,
  ADAPCC_ERR_INVALID_ARGUMENT = 1,
  ADAPCC_ERR_INVALID_STRATEGY = 2,
  ADAPCC_ERR_UNSUPPORTED = 3,
  ADAPCC_ERR_CUDA = 4,
  ADAPCC_ERR_BOOTSTRAP = 5,
  ADAPCC_ERR_OOM = 6,
  ADAPCC_ERR_TIMEOUT = 7,
  ADAPCC_ERR_MISMATCH = 8
} adapcc_result_t;

typedef enum { ADAPCC_FLOAT32 = 0, ADAPCC_BFLOAT16 = 1, ADAPCC_INT32 = 2 } adapcc_dtype_t;
typedef enum {
  ADAPCC_ALLREDUCE = 0, ADAPCC_ALLGATHER = 1, ADAPCC_ALLTOALL = 2,
  ADAPCC_REDUCE = 3, ADAPCC_BROADCAST = 4, ADAPCC_REDUCESCATTER = 5
} adapcc_coll_t;

/* Transport modes.  DIRECT: every rank's send/recv buffer is addressable by
 * the engine (loopback: one process owns all virtual ranks), so data moves
 * once from source to destination.  STAGED: a rank only touches its own
 * buffers plus the peers' IPC-mapped scratch arenas (landing and broadcast
 * slots with per-chunk flags) -- the multi-process protocol. */
typedef enum { ADAPCC_MODE_DIRECT = 0, ADAPCC_MODE_STAGED = 1 } adapcc_mode_t;

/* ACCUMULATE: recvbuf += result (one rounding), the paper's phase 2 in which
 * the late ranks' data is combined with the phase-1 result. */
#define ADAPCC_FLAG_ACCUMULATE 0x1u
/* Late join (a relay that becomes ready during phase 1 makes
 * "data chunks with the same offset in the buffer join the ongoing aggregation
 * process. Then in phase 2, only partial data chunks from relay workers that
 * have not been aggregated need to be broadcast").  AllReduce only, every
 * plan kind (loopback DIRECT / STAGED, multi-process STAGED via
 * adapcc_allreduce, zero-copy via adapcc_collective_zc); not combinable with
 * ACCUMULATE.  A non-ready rank passes its (future) sendbuf: it is read only
 * after the rank signalled ready (adapcc_signal_ready); it may not overlap
 * that rank's recvbuf (phase 1 writes the recvbuf before phase 2 reads the
 * chunks it missed) -- INVALID_ARGUMENT.
 *   LATE_JOIN (phase 1, mask R): every tree root also folds, per work piece
 *     (DIRECT) or per chunk (STAGED), the inputs of the non-ready ranks whose
 *     ready word already holds this call's ticket (appended after the
 *     regular sources, ascending rank), and records which ones it folded.
 *     DIRECT: the root reads the late input; STAGED: the late rank pushes its
 *     chunk to the root iff it is ready when its GPU reaches that chunk, and a
 *     per-chunk decision word next to the landing slot tells the root.
 *   LATE_COMPLEMENT (phase 2, SAME mask R and buffers as phase 1): recvbuf +=
 *     sum of the non-ready ranks' inputs that phase 1 did not fold, per piece /
 *     chunk (STAGED: only those chunks are pushed; the root broadcasts the sum
 *     of what was left, or a "nothing" decision, chunk by chunk).
 *     It complements the most recent LATE_JOIN call of the same plan (same
 *     strategy, count, dtype, mask and buffers kind); phase-1 / phase-2 pairs
 *     of different plans may interleave.  A second LATE_COMPLEMENT after the
 *     same phase 1 adds nothing.  No phase 1 of this plan yet: INVALID_ARGUMENT.
 * After both phases every rank holds the sum over all ranks. */
#define ADAPCC_FLAG_LATE_JOIN 0x2u
#define ADAPCC_FLAG_LATE_COMPLEMENT 0x4u

/* Bootstrap all-gather the caller implements (Python: torch.distributed
 * all_gather on the process group).  Gathers bytes_per_rank from every rank
 * into recv in rank order.  Returns 0 on success.  Used once in adapcc_init
 * to exchange CUDA IPC handles (the paper's "AllGather communication" of
 * IPC handles into a memory pointer table, §V-A, Fig. 10). */
typedef int (*adapcc_bootstrap_allgather_fn)(const void* send, void* recv,
                                             size_t bytes_per_rank, void* ctx);

/* ---------------------------------------------------------------- setup --- */

/* Multi-process communicator: one process per GPU (§V-A).
 * Allocates a scratch arena of scratch_bytes (0 = default 1 GiB) on
 * cuda_device, exports it with cudaIpcGetMemHandle, all-gathers the handles
 * through ag(), and maps every peer's arena.  Blocking; every rank must call
 * it.  Mode is STAGED.  Installs the default strategies. */
ADAPCC_API adapcc_result_t adapcc_init(adapcc_comm_t* comm, int rank, int nranks, int cuda_device,
                            size_t scratch_bytes, adapcc_bootstrap_allgather_fn ag,
                            void* ag_ctx);

/* Loopback communicator: nranks VIRTUAL ranks hosted by this process on one
 * device; one kernel launch executes every virtual rank's part of the
 * collective with the same engine and flag protocol (mode STAGED), or the
 * single-copy DIRECT plan.  scratch_bytes is per virtual rank. */
ADAPCC_API adapcc_result_t adapcc_init_loopback(adapcc_comm_t* comm, int nranks, int cuda_device,
                                     size_t scratch_bytes, adapcc_mode_t mode);

/* Replace the strategy of one collective (§IV-B/§VI-E graph reconstruction
 * without restart).  strategy_text: NUL-terminated,
 * format DESIGN.md §2; nranks in the text must equal the communicator's.
 * Takes effect for every later call in issue order; calls already enqueued
 * keep the strategy they were issued with (their plan tables stay alive).
 * stream is accepted for API symmetry; the swap itself needs no device work.
 * Errors: INVALID_STRATEGY (parse/validate), INVALID_ARGUMENT (coll). */
ADAPCC_API adapcc_result_t adapcc_set_strategy(adapcc_comm_t comm, adapcc_coll_t coll,
                                    const char* strategy_text, adapcc_stream_t stream);

/* ---------------------------------------------- collectives (multi-process) --- */

/* AllReduce (SUM) of count elements: every rank, relays included, receives
 * sum_{r ready} sendbuf_r in recvbuf.
 * ready_mask bit r = rank r is ready; bits >= nranks must be 0.
 * A non-ready rank's sendbuf is never read and may be NULL.
 * In place allowed (sendbuf == recvbuf).  flags: ADAPCC_FLAG_ACCUMULATE. */
ADAPCC_API adapcc_result_t adapcc_allreduce(adapcc_comm_t comm, const void* sendbuf, void* recvbuf,
                                 size_t count, adapcc_dtype_t dtype, uint64_t ready_mask,
                                 unsigned flags, adapcc_stream_t stream);

/* AllGather = one Broadcast per source: recvbuf holds nranks slots of
 * sendcount elements; slot s receives sendbuf_s for every ready s; slots of
 * non-ready sources are left untouched.  In place allowed when
 * sendbuf == recvbuf + rank*sendcount*esize. */
ADAPCC_API adapcc_result_t adapcc_allgather(adapcc_comm_t comm, const void* sendbuf, void* recvbuf,
                                 size_t sendcount, adapcc_dtype_t dtype, uint64_t ready_mask,
                                 adapcc_stream_t stream);

/* AlltoAll: sendbuf and recvbuf hold nranks
 * blocks of count_per_peer elements; block d of rank s lands in block s of
 * rank d, for every ready s.  Aliasing sendbuf/recvbuf is an error. */
ADAPCC_API adapcc_result_t adapcc_alltoall(adapcc_comm_t comm, const void* sendbuf, void* recvbuf,
                                size_t count_per_peer, adapcc_dtype_t dtype,
                                uint64_t ready_mask, adapcc_stream_t stream);

/* ---------------------------------------------------- collectives (loopback) --- */
/* Same semantics; sendbufs/recvbufs are HOST arrays of nranks device pointers,
 * one per virtual rank.  Non-ready entries of sendbufs may be NULL. */
ADAPCC_API adapcc_result_t adapcc_allreduce_lb(adapcc_comm_t comm, const void* const* sendbufs,
                                    void* const* recvbufs, size_t count, adapcc_dtype_t dtype,
                                    uint64_t ready_mask, unsigned flags, adapcc_stream_t stream);
ADAPCC_API adapcc_result_t adapcc_allgather_lb(adapcc_comm_t comm, const void* const* sendbufs,
                                    void* const* recvbufs, size_t sendcount,
                                    adapcc_dtype_t dtype, uint64_t ready_mask,
                                    adapcc_stream_t stream);
ADAPCC_API adapcc_result_t adapcc_alltoall_lb(adapcc_comm_t comm, const void* const* sendbufs,
                                   void* const* recvbufs, size_t count_per_peer,
                                   adapcc_dtype_t dtype, uint64_t ready_mask,
                                   adapcc_stream_t stream);

/* ------------------------------- more primitives on the same engine (NEXT-4) ---
 * Reduce: the root receives sum_{r ready} sendbuf_r (the paper's Reduce, whose
 * strategy AllReduce reverses; evaluated in Fig. 11).
 * Every tree of a Reduce strategy is rooted at `root` (else INVALID_ARGUMENT);
 * without a user strategy a star rooted at `root` is used.  Only the root's
 * recvbuf is written (non-roots may pass NULL).  flags: ACCUMULATE.
 * Broadcast: every rank's recvbuf receives the root's sendbuf;
 * nothing is written when the root is not ready.  In place at the root allowed.
 * ReduceScatter: rank b receives block b (recvcount elements) of
 * sum_{r ready} sendbuf_r, reduced along the "rtree dst=b" lines of the
 * strategy (default: a star rooted at b).  sendbuf holds nranks blocks; in
 * place allowed when recvbuf == sendbuf + rank*recvcount*esize. */
ADAPCC_API adapcc_result_t adapcc_reduce(adapcc_comm_t comm, const void* sendbuf, void* recvbuf,
                                         size_t count, adapcc_dtype_t dtype, int root,
                                         uint64_t ready_mask, unsigned flags, adapcc_stream_t stream);
ADAPCC_API adapcc_result_t adapcc_broadcast(adapcc_comm_t comm, const void* sendbuf, void* recvbuf,
                                            size_t count, adapcc_dtype_t dtype, int root,
                                            uint64_t ready_mask, adapcc_stream_t stream);
ADAPCC_API adapcc_result_t adapcc_reducescatter(adapcc_comm_t comm, const void* sendbuf, void* recvbuf,
                                                size_t recvcount, adapcc_dtype_t dtype,
                                                uint64_t ready_mask, unsigned flags,
                                                adapcc_stream_t stream);
ADAPCC_API adapcc_result_t adapcc_reduce_lb(adapcc_comm_t comm, const void* const* sendbufs,
                                            void* const* recvbufs, size_t count, adapcc_dtype_t dtype,
                                            int root, uint64_t ready_mask, unsigned flags,
                                            adapcc_stream_t stream);
ADAPCC_API adapcc_result_t adapcc_broadcast_lb(adapcc_comm_t comm, const void* const* sendbufs,
                                               void* const* recvbufs, size_t count,
                                               adapcc_dtype_t dtype, int root, uint64_t ready_mask,
                                               adapcc_stream_t stream);
ADAPCC_API adapcc_result_t adapcc_reducescatter_lb(adapcc_comm_t comm, const void* const* sendbufs,
                                                   void* const* recvbufs, size_t recvcount,
                                                   adapcc_dtype_t dtype, uint64_t ready_mask,
                                                   unsigned flags, adapcc_stream_t stream);

/* AlltoAllv (NEXT-4; skewed MoE token dispatch): counts is a
 * HOST array of nranks*nranks element counts, counts[s*nranks + d] from rank s
 * to rank d, identical on every rank.  Rank s's sendbuf holds its blocks in
 * destination order, rank d's recvbuf its blocks in source order (packed).
 * Blocks from non-ready sources are left untouched.  The a2a lines of the
 * AlltoAll strategy split every block by weight. */
ADAPCC_API adapcc_result_t adapcc_alltoallv(adapcc_comm_t comm, const void* sendbuf, void* recvbuf,
                                            const uint64_t* counts, adapcc_dtype_t dtype,
                                            uint64_t ready_mask, adapcc_stream_t stream);
ADAPCC_API adapcc_result_t adapcc_alltoallv_lb(adapcc_comm_t comm, const void* const* sendbufs,
                                               void* const* recvbufs, const uint64_t* counts,
                                               adapcc_dtype_t dtype, uint64_t ready_mask,
                                               adapcc_stream_t stream);

/* ----------------------------------------------- zero-copy (multi-process) ---
 * Register a device buffer so that peers can read/write it directly: the
 * allocation holding [ptr, ptr+bytes) is exported with CUDA IPC and mapped by
 * every peer (one bootstrap all-gather; the paper's IPC "memory pointer
 * table").  Collective: every rank registers a buffer of the same size
 * in the same order; ids are assigned in that order.  The buffer must stay
 * allocated until adapcc_deregister_buffer (collective, synchronizes the
 * device).  UNSUPPORTED on loopback communicators (already zero-copy).
 * adapcc_collective_zc runs any collective on registered buffers with the
 * single-copy DIRECT plan across processes: a tree's root reads every rank's
 * input slice straight from its registered sendbuf and writes the result
 * straight into every rank's registered recvbuf over NVLink -- no landing or
 * broadcast slots -- bracketed by in-kernel entry/exit barriers.  Offsets
 * (bytes, multiples of 16) and count must be identical on every rank; count
 * has the same meaning as in the collective's own entry point. */
ADAPCC_API adapcc_result_t adapcc_register_buffer(adapcc_comm_t comm, void* ptr, size_t bytes,
                                                  int* reg_id);
ADAPCC_API adapcc_result_t adapcc_deregister_buffer(adapcc_comm_t comm, int reg_id);
ADAPCC_API adapcc_result_t adapcc_collective_zc(adapcc_comm_t comm, adapcc_coll_t coll, int send_reg,
                                                size_t send_offset, int recv_reg, size_t recv_offset,
                                                size_t count, adapcc_dtype_t dtype, int root,
                                                uint64_t ready_mask, unsigned flags,
                                                adapcc_stream_t stream);

/* NVLS switch reduction (NEXT-2): set up a multicast team over every rank's
 * GPU (NVSwitch multicast objects, cuMulticast*) bound to `bytes` (rounded
 * up to the multicast granularity) of library-owned scratch per rank; after
 * it AllReduce strategies may contain `nvls weight=<w> chunk=<C>` lines,
 * whose partition every rank copies into its scratch, slice owners sum in
 * the switch (multimem.ld_reduce) and store to every rank at once
 * (multimem.st), and every rank copies out -- ~S per GPU and direction over
 * NVLink instead of the 2(n-1)/n S of P2P trees.  The switch defines the fp32
 * summation order (oracle: tolerance mode, int32 exact); nvls lines need the
 * whole ready mask and no late join (UNSUPPORTED otherwise) and run on the
 * LDG kernel.  Collective over every rank.  Loopback (one device, no
 * multicast team): the switch is EMULATED -- each virtual rank gets its own
 * scratch and the kernel sums the n copies in ascending rank order and
 * stores the sum to all of them, so the plan (copy in, per-slice flags,
 * switch step, copy out, ragged tail) runs and is tested on one GPU; only
 * multimem itself is not exercised there.  Multi-process: any failure on any
 * rank (no multicast support, driver entry
 * points, pidfd_getfd of rank 0's exported handle, binding) makes every rank
 * return UNSUPPORTED and `why` (may be NULL) says why; an nvls line then
 * makes its calls return UNSUPPORTED.  Calling it again replaces the team.
 * Off by default. */
ADAPCC_API adapcc_result_t adapcc_nvls_setup(adapcc_comm_t comm, size_t bytes, char* why, size_t why_len);

/* Ticket of the most recent LATE_JOIN call (0 before the first). */
ADAPCC_API adapcc_result_t adapcc_late_ticket(adapcc_comm_t comm, uint64_t* ticket);
/* Consume a ticket without a LATE_JOIN call (host only; collective in the
 * sense that every rank must advance at the same point of its call
 * sequence): a coordinator that runs a plain AllReduce because everyone was
 * ready still retires the readiness signals of that round.  *ticket (may be
 * NULL) = the consumed ticket. */
ADAPCC_API adapcc_result_t adapcc_late_advance(adapcc_comm_t comm, uint64_t* ticket);

/* Link probe (NEXT-2: the paper's alpha-beta link profiling, §IV-B,
 * P:L109-115).  Rank `src` (-1 = this rank; loopback: any virtual rank) sends
 * `messages` back-to-back messages of `bytes` (multiple of 16, > 0, at most
 * one parity half's data region) to EVERY rank in dst_mask at once, through
 * engine 0 (copy engines: cudaMemcpyAsync, one stream per destination) or 1
 * (SM: TMA bulk copies global -> shared -> peer, one kernel per message).
 * `iters` repetitions are captured in one CUDA graph, replayed once (warm-up)
 * and once between CUDA events; *seconds = that time / iters, the mean time of
 * one repetition (so a repetition of m messages of s bytes is the paper's
 * t = m (alpha + beta s), with no host launch cost inside).
 * Data goes from the sender's arena (half 0) to the receivers' arenas (half 1):
 * the call first synchronizes the device, and in multi-process mode it is a
 * collective -- every live rank calls it (with its own src / dst_mask, 0 =
 * only take part) and the timed replays start after a bootstrap barrier, so
 * a probe round of the Fig. 5(b) schedule runs all its flows at once.
 * dst_mask must not contain src or excluded ranks.  Errors: INVALID_ARGUMENT,
 * CUDA, BOOTSTRAP. */
ADAPCC_API adapcc_result_t adapcc_link_probe(adapcc_comm_t comm, int src, uint64_t dst_mask, size_t bytes,
                                             int messages, int engine, int iters, double* seconds);
/* Mark `rank` ready for late join: after all prior work on `stream` (e.g. the
 * rank's gradient computation) its ready word becomes `ticket` (0 = the
 * current ticket).  Multi-process: rank must be this rank (or -1);
 * loopback: any virtual rank. */
ADAPCC_API adapcc_result_t adapcc_signal_ready(adapcc_comm_t comm, int rank, uint64_t ticket,
                                               adapcc_stream_t stream);

/* Readiness board (NEXT-1 online coordinator): a page of host
 * memory, mapped into the device, whose word r holds the ticket rank r last
 * signalled ready for -- adapcc_signal_ready's kernel writes it (system-scope
 * release) next to the arena word, so a host thread can poll readiness at a
 * microsecond cycle without touching the device.  Words 64..127 are free for
 * the coordinator's own use (its decision channel).  *shared = 1 when every
 * rank's word is visible on this host: always in loopback; in multi-process
 * mode when the ranks share a node and POSIX shared memory works (the page is
 * created by rank 0 at adapcc_init and mapped by every rank); 0 = only this
 * rank's word is maintained.  The page lives until adapcc_finalize. */
ADAPCC_API adapcc_result_t adapcc_ready_board(adapcc_comm_t comm, volatile uint64_t** board, int* shared);
/* Benchmark utility: one thread spins on %globaltimer for `ns` nanoseconds on
 * `stream` (the controlled straggler of SURVEY §8(d) d-5: a late rank's
 * "computation" that occupies one SM slot, not the GPU). */
ADAPCC_API adapcc_result_t adapcc_spin(adapcc_comm_t comm, uint64_t ns, adapcc_stream_t stream);

/* Online coordinator, native decision loops (NEXT-1 / NEXT-3; host only, no
 * device work, callable without a GPU).  `board` is the page
 * adapcc_ready_board returns (or any >= 64-word array laid out the same way:
 * word r = the ticket rank r last signalled).  Times are CLOCK_MONOTONIC
 * seconds (the clock of Python's time.perf_counter on Linux).  Both loops
 * spin on plain host loads and return without touching the communicator, so
 * a binding may call them with its interpreter lock released.
 *
 * adapcc_coord_decide -- the break-even (ski-rental) rule of P:L133-137 on
 * real readiness.  Every cycle_s it reads which ranks in `members` have
 * signalled `ticket`: all of them -> *full = 1, *ready_mask = members; else,
 * with k >= 1 ready, if the time already waited (cycles x cycle_s) plus one
 * more cycle exceeds buy_cost[k] (the estimated phase-1 + phase-2 time with k
 * ready ranks; array of nranks + 1 doubles) -> *full = 0,
 * *ready_mask = the ready ranks (phase 1); else wait one more cycle.
 * *t_first = when the first rank was seen ready (T_fault's origin),
 * *t_decide = when the decision was taken.  Errors: INVALID_ARGUMENT,
 * TIMEOUT (nobody ready within timeout_s).
 *
 * adapcc_coord_await -- after phase 1 was enqueued: wait until every rank in
 * late_mask has signalled `ticket` (*faulty = 0: run phase 2) or, with
 * fault_factor > 0, until T_fault = fault_factor x (phase-1 end - t_first)
 * has passed since phase 1 ended (*faulty = the late ranks still not ready,
 * P:L139).  Phase 1's end is when `phase1_event` (a cudaEvent_t recorded after
 * it; NULL = already ended) first reports complete.  Errors:
 * INVALID_ARGUMENT, CUDA (event query failed), TIMEOUT (timeout_s passed). */
ADAPCC_API adapcc_result_t adapcc_coord_decide(const volatile uint64_t* board, int nranks, uint64_t members,
                                               uint64_t ticket, const double* buy_cost, double cycle_s,
                                               double timeout_s, uint64_t* ready_mask, int* full,
                                               double* t_first, double* t_decide);
ADAPCC_API adapcc_result_t adapcc_coord_await(const volatile uint64_t* board, int nranks, uint64_t late_mask,
                                              uint64_t ticket, void* phase1_event, double t_first,
                                              double fault_factor, double timeout_s, uint64_t* faulty);

/* ------------------------------------------------------------- lifecycle --- */

/* Latched device error (TIMEOUT) or SUCCESS.  Does not synchronize. */
ADAPCC_API adapcc_result_t adapcc_get_async_error(adapcc_comm_t comm);
/* NEXT-3 fault tolerance ("the coordinator identifies the
 * remaining non-ready workers as faulty workers ... excluded from the training
 * group"; "graph reconstruction" without restarting the job).
 * Survivors exclude the ranks in dead_mask and keep the communicator: arenas,
 * IPC mappings and registered buffers stay; a latched TIMEOUT is cleared; the
 * device epoch restarts above every flag posted so far; every collective's
 * strategy is reset to the survivors' default (AllReduce: one star per live
 * rank).  Afterwards excluded ranks are never ready, own no work, and none of
 * their buffers or arena bytes is read or written; set_strategy accepts a
 * strategy that names them only as tree leaves (not AlltoAll relays, Reduce
 * roots or Broadcast sources).  Collective over the SURVIVORS: each calls it
 * with the same dead_mask and an all-gather `ag` over exactly the survivors
 * (ascending rank order; ag may be NULL in loopback).  Host-blocking: waits for
 * this device to drain.  Precondition: the excluded ranks' GPU work has stopped
 * (their launches exit at the watchdog deadline).  CUDA graphs captured before
 * the call must not be replayed after it.  Multi-process: every later launch
 * also runs the debug call check's start barrier (all survivors' kernels of a
 * launch have started and make the same call before any byte moves; see
 * "debug_check" and DESIGN.md §12, known issue).  INVALID_ARGUMENT: bits >= nranks,
 * nothing left alive, or (multi-process) this rank excluded / ag NULL. */
ADAPCC_API adapcc_result_t adapcc_exclude(adapcc_comm_t comm, uint64_t dead_mask,
                               adapcc_bootstrap_allgather_fn ag, void* ag_ctx);

/* Live ranks (all ranks until adapcc_exclude). */
ADAPCC_API adapcc_result_t adapcc_members(adapcc_comm_t comm, uint64_t* members);

/* Synchronizes the device, unmaps peers, frees everything.  comm may be NULL. */
ADAPCC_API adapcc_result_t adapcc_finalize(adapcc_comm_t comm);
ADAPCC_API const char* adapcc_strerror(adapcc_result_t r);
/* Text of the CUDA error behind the calling thread's last ADAPCC_ERR_CUDA. */
ADAPCC_API const char* adapcc_last_cuda_error(void);

/* Runtime knobs.  key: "timeout_ms" (watchdog, default 10000; env
 * ADAPCC_TIMEOUT_MS), "max_ctas" (grid cap, 0 = #SMs x occupancy; env
 * ADAPCC_NCTAS; a change empties the plan cache, since pieces are sized for the grid), "engine" (2 = auto by call size, default:
 * the LDG fold below 128 MiB of traffic per launch, the TMA pipeline above, and ACCUMULATE plans
 * without flags or arena streams under 32 MiB the flat kernel; 1 = TMA bulk-copy pipeline; 0 = 128-bit
 * LDG/STG fold; 3 = flat kernel for every plan without flags, arena streams, late join or NVLS
 * (others keep the auto choice): the whole grid strides through all tasks' vectors, no work items;
 * env ADAPCC_ENGINE), "flat_ctas" (flat kernel grid: CTAs per SM, 1..64, default 2 = resident;
 * env ADAPCC_FLAT_CTAS), "piece_kib" (traffic per work
 * piece of flag-free tasks, 0 = automatic, default; env ADAPCC_PIECE_KIB), "taper" (the last
 * ~2 x grid flag-free items are cut into this many sub-pieces, 0..64; 0 = automatic,
 * default: halve those of >= 384 KiB of traffic; 1 = off;
 * env ADAPCC_TAPER), "sched" (LDG fold kernel: 0 = CTAs claim items from a counter; 1 or 2 =
 * static schedule, default: CTA b runs items b, b + grid, ... and prefetches each item's
 * descriptor blob while it folds the previous one -- plans whose blobs exceed 64 MiB claim
 * dynamically; env ADAPCC_SCHED), "pdl" (1 = launch engine kernels as programmatic dependent
 * launches: a kernel's prologue overlaps the previous kernel on the stream, default; 0 = off;
 * env ADAPCC_PDL), "first_blob" (LDG fold kernel: 1 = item descriptors as per-item blobs,
 * default; 0 = plain item/task/ref tables; env ADAPCC_FIRST_BLOB; env only: ADAPCC_TMA_SHAPE
 * forces the TMA ring of every TMA launch, 1 = 1 CTA/SM x 3 x 64 KiB, 2 = 2 CTAs/SM x 3 x 32 KiB,
 * 0 = automatic, default: STAGED plans (and ACCUMULATE plans with acc_red off) 2, others 1),
 * "default_chunk" (chunk C_m in bytes of every default strategy -- the ones in effect for collectives
 * without adapcc_set_strategy; multiple of 16, default 262144; e.g. the cost model's choice from
 * a link profile, costmodel.py; strategies set by the caller are kept),
 * "acc_red" (TMA kernel, accumulating destinations -- ACCUMULATE phase 2, LATE_COMPLEMENT: 1 = the
 * folded tile leaves the stage by TMA bulk reduce-adds, recv += result performed in L2
 * (cp.reduce.async.bulk .add, fp32 / bf16 round to nearest even without flushing subnormals,
 * int32 wraps), default; 0 = recv tiles are TMA-loaded into the stage, added in shared memory
 * and bulk-stored; env ADAPCC_ACC_RED; a change empties the plan cache), "trace" (in-kernel trace capacity in
 * records, 0 = off, default; see adapcc_trace_read), "debug_check" (multi-process: 1 = every launch first compares a hash
 * of its call -- collective, strategy, count, dtype, mask, flags, live ranks, segment, zero-copy
 * registrations -- with every live peer's for the same launch, in the arena headers, before any
 * byte moves; a mismatch latches ADAPCC_ERR_MISMATCH instead of corrupting data or hanging until
 * the watchdog; 0 = off, default; env ADAPCC_DEBUG), "debug_drop_rank" (loopback test hook:
 * virtual rank r posts nothing, so its consumers hit the watchdog; -1 = off).  Changing engine / piece_kib / taper / sched / first_blob empties the
 * plan cache (plans a captured CUDA graph uses stay alive); results never depend on them. */
ADAPCC_API adapcc_result_t adapcc_config(adapcc_comm_t comm, const char* key, int64_t value);

/* In-kernel trace (debug / tuning; SURVEY §5 tracing).  Enable with adapcc_config(comm, "trace",
 * capacity) -- capacity = records kept (0 = off, the default; changing it drains the device and
 * drops the old buffer).  While on, every engine launch appends one 48-byte record per work item
 * it executes and one per CTA, with %globaltimer times in ns:
 *   struct { uint32_t launch, cta, item, task; uint64_t t0, t1, t2, bytes; }
 *   item record (item != 0xFFFFFFFF): t0 claimed, t1 inputs ready (flags acquired), t2 done
 *     (stores issued, flags posted); bytes = traffic of the item over all its streams;
 *   CTA record (item == 0xFFFFFFFF): t0 entry, t1 after the stream-order wait and epoch read,
 *     t2 exit.
 * Records beyond the capacity are dropped.  adapcc_trace_read drains the device, copies up to
 * max_records records to host memory `records`, reports how many were copied and how many were
 * written in total (n_total > capacity: some were dropped), and empties the buffer.  Returns
 * ADAPCC_ERR_UNSUPPORTED while tracing is off.  Tracing adds one atomic per record. */
ADAPCC_API adapcc_result_t adapcc_trace_read(adapcc_comm_t comm, void* records, uint32_t max_records,
                                             uint32_t* n_copied, uint32_t* n_total);

/* Number of engine kernel launches this communicator has issued. */
ADAPCC_API adapcc_result_t adapcc_launch_count(adapcc_comm_t comm, uint64_t* count);
/* Kernel of the most recent launch: 0 = LDG/STG fold, 1 = TMA pipeline, 3 = flat kernel, -1 = none. */
ADAPCC_API adapcc_result_t adapcc_last_engine(adapcc_comm_t comm, int* engine);

/* ------------------------------------------------- host-only inspection ---
 * No GPU needed.  Used by the CPU tests to cross-check the C++ loader and
 * planner against the oracle (they share no code). */

/* Parse + validate.  On success fills nranks, coll, nsubs (after ring
 * expansion); on INVALID_STRATEGY writes a message into err (may be NULL). */
ADAPCC_API adapcc_result_t adapcc_strategy_check(const char* strategy_text, int* nranks, int* coll,
                                      int* nsubs, char* err, size_t err_len);

/* Behaviour tuples of sub-collective `sub` under ready_mask:
 * tuples[4*g + {0,1,2,3}] = isActive, hasRecv, hasKernel, hasSend of rank g;
 * nflows[g] = number of flows rank g emits upward (Fig. 8(b)). */
ADAPCC_API adapcc_result_t adapcc_strategy_tuples(const char* strategy_text, int sub, uint64_t ready_mask,
                                       uint8_t* tuples, int32_t* nflows);

/* Effective integer weight, chunk bytes, parent array and bcast source of
 * sub-collective `sub` (parent: nranks entries, -1 at the root). */
ADAPCC_API adapcc_result_t adapcc_strategy_sub(const char* strategy_text, int sub, int64_t* weight,
                                    int64_t* chunk_bytes, int32_t* parent, int32_t* src);

/* Route of AlltoAll flow src -> dst in a2a sub-collective `sub` (routing
 * variables x^f_ij, eq. 1; DESIGN.md §2 `route=`): writes the relay
 * ranks in path order into hops (capacity nranks entries) and their number
 * into *nhops (0 = direct).  INVALID_ARGUMENT for a non-a2a sub or ranks out
 * of range.  Host-only. */
ADAPCC_API adapcc_result_t adapcc_strategy_route(const char* strategy_text, int sub, int src, int dst,
                                      int32_t* hops, int* nhops);

/* Partition (DESIGN.md §3 Q9): bounds[0..nsubs] of `count` elements over all
 * sub-collectives (allreduce/alltoall), or over the bcast lines of source
 * `src` (allgather; bounds has (#lines of src)+1 entries). */
ADAPCC_API adapcc_result_t adapcc_strategy_partition(const char* strategy_text, uint64_t count,
                                          adapcc_dtype_t dtype, int src, uint64_t* bounds,
                                          int* nbounds);

/* Plan statistics for one rank (-1 = all virtual ranks) of a call, with the
 * live-rank set `members` (0 = all ranks; see adapcc_exclude): INVALID_STRATEGY
 * if the strategy gives an excluded rank work, INVALID_ARGUMENT if the ready
 * mask names one. */
typedef struct {
  uint64_t tasks;         /* fold/copy tasks */
  uint64_t items;         /* (task, chunk) work items */
  uint64_t levels;        /* dependency depth + 1 */
  uint64_t segments;      /* launches the call is split into */
  uint64_t bytes_read;    /* payload bytes loaded by the engine */
  uint64_t bytes_written; /* payload bytes stored by the engine */
  uint64_t remote_bytes;  /* of which cross a rank boundary (loads+stores) */
  uint64_t arena_bytes;   /* scratch bytes used per rank (max over ranks) */
} adapcc_plan_stats_t;

ADAPCC_API adapcc_result_t adapcc_plan_stats(const char* strategy_text, uint64_t count,
                                  adapcc_dtype_t dtype, uint64_t ready_mask, unsigned flags,
                                  adapcc_mode_t mode, int rank, size_t scratch_bytes,
                                  uint64_t members, adapcc_plan_stats_t* stats);

/* Host-only inspection of the work items the engine would execute for one segment (launch) of a
 * call: the plan compiler's output (DESIGN.md §6 "Work items", "Pieces"), for CPU tests of the
 * host logic.  grid = CTAs of the launch (pieces are sized for it), tma = 1 for the TMA pipeline's
 * piece rule, piece_kib / taper as adapcc_config (0 = automatic).  Items come in claim order; an
 * item covers elements [off, off + len) of chunk `chunk` of task `task` (element offsets from the
 * chunk start).  Tasks are listed with their element range, chunking, stream counts, flag counts
 * and dependency level.  Up to max_items / max_tasks entries are copied; *n_items / *n_tasks get
 * the full counts.  segment >= the number of segments: INVALID_ARGUMENT. */
typedef struct { uint32_t task, chunk, off, len; } adapcc_item_t;
typedef struct {
  uint64_t lo, hi;                  /* elements covered */
  uint32_t chunk_elems, nchunks;
  uint16_t nsrc, ndst, nwait, npost;
  uint32_t level;                   /* dependency depth: waits only on posts of lower levels */
  uint32_t owner;                   /* executing rank */
} adapcc_task_info_t;
ADAPCC_API adapcc_result_t adapcc_plan_items(const char* strategy_text, uint64_t count,
                                  adapcc_dtype_t dtype, uint64_t ready_mask, unsigned flags,
                                  adapcc_mode_t mode, int rank, size_t scratch_bytes, int grid,
                                  int tma, uint32_t piece_kib, int taper, int segment,
                                  adapcc_item_t* items, uint32_t max_items, uint32_t* n_items,
                                  adapcc_task_info_t* tasks, uint32_t max_tasks, uint32_t* n_tasks);

#ifdef __cplusplus
}
#endif

#endif /* ADAPCC_H */
