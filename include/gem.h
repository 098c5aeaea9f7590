/* gem.h -- C ABI of libgem, the B200 (sm_100a) GEM VLIW interpreter.
 *
 * The operation (§II): a netlist compiled into an
 * executable simulator is run with input stimuli, cycle by cycle, producing
 * outputs; speed is measured in simulated cycles per second.  Simulation is
 * oblivious/full-cycle, synchronous and 2-state.
 * The compiled form is the VLIW "bitstream" of §III-E produced by
 * the mapper (gem_map.h); each thread block interprets one partition's
 * program per cycle and blocks synchronise at stage and cycle
 * boundaries.
 *
 * Conventions
 *  - All functions return 0 (GEM_OK) or a negative GEM_E_* code; no C++
 *    exception crosses the ABI.  gem_last_error() returns a thread-local
 *    message for the last failure.
 *  - Bit order: signal i of a vector is bit i%32 of word i/32; the last word
 *    is zero-padded.
 *  - PI order = AIGER input order with RAM rdata inputs removed; PO and flop
 *    order = AIGER output / latch order.  (Internally the mapper permutes flops
 *    and POs into partition-owned words; every call below speaks external order.)
 *  - Ownership: the library copies caller buffers and never retains caller
 *    pointers.  Host pointers are plain pageable or pinned memory; pointers
 *    flagged *_on_device are CUDA device pointers on the handle's device.
 *  - Threading: a handle is not re-entrant.  Handles on different devices are
 *    independent.
 *  - A CUDA error is sticky: the handle is poisoned (GEM_E_CUDA) and only
 *    gem_free() is valid afterwards.
 */
#ifndef GEM_H
#define GEM_H
#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define GEM_OK 0
#define GEM_E_INVAL -1        /* null pointer, size mismatch, bad argument        */
#define GEM_E_FORMAT -2       /* bad magic / version / truncated program blob     */
#define GEM_E_CUDA -3         /* CUDA failure; handle poisoned                    */
#define GEM_E_NOMEM -4        /* device allocation failed                          */
#define GEM_E_NOINPUT -5      /* gem_step(n) with fewer than n queued input cycles */
#define GEM_E_UNSUPPORTED -6  /* e.g. no CUDA device, co-residency impossible      */

/* gem_config.flags (parity instruments; both off in timed runs) */
#define GEM_F_TRACE_STATE 0x1u  /* record Q(t+1) every cycle (gem_read_state_trace) */
#define GEM_F_DIGEST 0x2u       /* record the per-cycle flop digest d_t              */
#define GEM_F_ASYNC 0x4u        /* gem_step returns without synchronising            */
#define GEM_F_PROFILE 0x8u      /* record per-CTA clock64 phase stamps (first 256 cycles) */
/* Activity-based pruning (the paper's next step, P:237-241:
 * "skip partitions whose inputs did not change").  A partition whose input-port
 * words (PI[t], Q_cur, RD_cur, stage cuts) equal those of the previous cycle
 * produces the same endpoint words, so its layers are skipped and its last
 * results are committed again; RAM ports still operate every cycle.  Results
 * are identical with and without the flag.  Applies to the bit-packed path for
 * CTAs that run one partition of one stream per stage and cycle (every
 * single-stream launch whose grid covers the partitions); other CTAs, and lane
 * mode, always evaluate.  The first cycle of every gem_step evaluates. */
#define GEM_F_ACTIVITY 0x10u
/* Launch-mode overrides (tests and measurements; results are identical):
 *   GEM_F_NO_RESIDENT  stream every program chunk through the TMA ring (no
 *                      shared-memory residency, no pinned prefix);
 *   GEM_F_NO_LANES     batched streams on the bit-packed path (no lane mode);
 *   GEM_F_STATIC_LANES lane mode with static LPT work lists instead of the
 *                      dynamic (ticketed) distribution. */
#define GEM_F_NO_RESIDENT 0x20u
#define GEM_F_NO_LANES 0x40u
#define GEM_F_STATIC_LANES 0x80u
/* Word mode (blobs mapped with words=1, gem_isa.h "WRD1"): runs with fewer
 * than 32 streams (or with GEM_F_NO_LANES) execute the partition's AND list
 * one signal per shared-memory word in barrier-separated steps instead of
 * bit-packed boomerang layers (the latency path); chosen
 * when every program a CTA runs fits in its shared memory, else the
 * bit-packed path runs.  Results are identical.  GEM_F_NO_WORDS keeps the
 * bit-packed path; GEM_F_ACTIVITY and split designs (dist_world > 1) always
 * use it. */
#define GEM_F_NO_WORDS 0x100u
/* (GEM_F_NO_RESIDENT applies to the bit-packed path; word programs are always
 * resident in shared memory.) */

typedef struct gem_sim gem_sim; /* opaque, owned by the library */

typedef struct {
  int device;           /* CUDA device ordinal                                     */
  uint32_t n_streams;   /* independent stimulus streams over the same design (>=1) */
  void* cuda_stream;    /* cudaStream_t to launch on, or NULL for a private stream */
  uint32_t flags;       /* GEM_F_*                                                 */
  uint32_t grid_limit;  /* 0 = auto (co-resident persistent grid); else max CTAs   */
  /* Launch tuning (0 = automatic; none of these changes results, only speed).
   * Bit-packed path: */
  uint32_t ctas_per_sm;      /* CTAs per SM (1..4)                                   */
  uint32_t max_group;        /* max streams sharing one work item (1..15)            */
  /* Lane mode (batched streams): */
  uint32_t lane_groups;      /* 32-stream groups per work item K (1, 2 or 4)          */
  uint32_t lane_ctas_per_sm; /* CTAs per SM (1 or 2)                                  */
  uint32_t lane_run;         /* work items per scheduling unit                        */
  /* L2 residency of streamed program chunks: fraction kept evict_last
   * (0 = automatic: a share of the L2 for programs larger than half of it;
   * > 0 = that fraction; < 0 = no eviction policy). */
  float l2_evict_last;
  /* Single-design multi-GPU (§V P:247 future work):
   * the design's partitions are split over dist_world devices (0 or 1 = one
   * device), this handle runs those owned by dist_rank (gem_dist_owner).  The
   * handle stays unusable for gem_step until gem_dist_connect. */
  uint32_t dist_world;
  uint32_t dist_rank;
} gem_config;

typedef struct {
  uint32_t n_pi, n_po, n_flops, n_rams, n_parts, n_stages, max_layers, total_layers;
  uint32_t pi_words, po_words, q_words;   /* external word counts per cycle/stream */
  uint32_t grid, blocks_per_sm, smem_bytes, n_streams;
  uint32_t resident;     /* CTAs whose programs all live in their shared memory */
  uint32_t ring_slots;   /* else: TMA ring depth used to stream program chunks */
  uint32_t group;        /* streams per work item (program chunks reused across them) */
  uint32_t lanes;        /* 1 = stream-sliced lane mode (32 streams per lane word)  */
  uint32_t words;        /* 1 = word mode (single-stream latency path, WRD1)        */
  uint64_t n_and;                          /* live 2-input ANDs (gate evals/cycle) */
  uint64_t n_and_mapped;                   /* with RepCut replication              */
  uint64_t program_bytes;
  uint64_t cycle;                          /* cycles simulated so far              */
} gem_info;

/* Compile step's output -> executable simulator (§II P:41 "compile
 * [the netlist] into an executable simulator"; §III-E P:178-196 the bitstream).
 * blob: host memory, nbytes bytes, the .gemb of gem_map.h; copied, not retained.
 * Allocates device state for cfg->n_streams independent streams: flops start at
 * their AIGER init values (uninitialised latches at 0, reading U5), RAM read
 * registers and RAM contents at 0 (U10).  *out receives the handle (NULL on
 * failure).  Errors: GEM_E_INVAL (null/size/n_streams 0/bad device),
 * GEM_E_FORMAT (bad magic, version, truncated or inconsistent tables),
 * GEM_E_UNSUPPORTED (no CUDA device; state or program ring does not fit in
 * shared memory; a partition with more than GEM_MAX_CHUNKS-2 layers),
 * GEM_E_NOMEM, GEM_E_CUDA.  On failure nothing is leaked. */
int gem_load_program(const void* blob, size_t nbytes, const gem_config* cfg, gem_sim** out);

/* Static facts of the loaded program and the chosen launch (host struct). */
int gem_info_get(const gem_sim* sim, gem_info* out);

/* Input stimuli ("executes it with input stimuli", one PI vector per
 * cycle applied before that cycle's evaluation, reading U12).
 * pi_words = uint32 [n_streams][ncycles][pi_words], PI order as above.
 * Replaces any inputs not yet consumed.  Host buffers: copied before return
 * (the caller may reuse the buffer, pinned or not, immediately).
 * src_on_device = 1 (a deviation from SURVEY §8(b), which has host buffers
 * only): pi_words is a device pointer on the handle's device, copied
 * asynchronously on the handle's stream (the caller keeps it alive until the
 * next gem_step has been enqueued).  Errors: GEM_E_INVAL (null with
 * ncycles > 0, ncycles > 2^32-16), GEM_E_NOMEM, GEM_E_CUDA. */
int gem_set_inputs(gem_sim* sim, const uint32_t* pi_words, uint64_t ncycles, int src_on_device);

/* Simulate ncycles clock cycles (cycle by cycle, synchronous,
 * 2-state; oblivious full-cycle evaluation P:46) with one persistent
 * cooperative kernel launch: per cycle and stage, every partition reads its
 * input ports once, runs its boomerang layers, commits flops,
 * POs and RAM ports, then a grid barrier.  Consumes
 * ncycles queued input vectors.  After return (or, with GEM_F_ASYNC, after the
 * stream reaches it) the state is Q[t0+ncycles].  ncycles = 0 is a no-op.
 * Errors: GEM_E_NOINPUT (fewer than ncycles queued), GEM_E_CUDA (including a
 * grid-barrier watchdog trap, reported in gem_last_error; handle poisoned). */
int gem_step(gem_sim* sim, uint64_t ncycles);

/* Outputs ("producing output"): PO[t0 .. t0+ncycles-1] of the last
 * gem_step, each sampled after the cycle's combinational evaluation and before
 * its clock edge (reading U11): uint32 [n_streams][ncycles][po_words], AIGER
 * output order.  dst: host memory, or a device pointer if dst_on_device
 * (the multi-GPU gather reads straight into a torch CUDA tensor).  Synchronous.
 * Errors: GEM_E_INVAL (null dst, ncycles > cycles of the last step). */
int gem_read_outputs(gem_sim* sim, uint32_t* po_words, uint64_t ncycles, int dst_on_device);

/* Flop state Q (the only state besides RAMs): uint32 [n_streams][q_words],
 * AIGER latch order; read after the last step, written before the next one
 * (checkpoint / resume).  Host or device buffers as flagged.
 * Synchronous.  Errors: GEM_E_INVAL (null). */
int gem_read_state(gem_sim* sim, uint32_t* flop_words, int dst_on_device);
int gem_write_state(gem_sim* sim, const uint32_t* flop_words, int src_on_device);

/* Parity instrument (SURVEY §8(c) protocol), needs GEM_F_TRACE_STATE: Q(t+1)
 * for every cycle of the last step, uint32 [n_streams][ncycles][q_words]
 * (host).  Errors: GEM_E_INVAL (flag not set, ncycles too large). */
int gem_read_state_trace(gem_sim* sim, uint32_t* dst, uint64_t ncycles);

/* Parity instrument, needs GEM_F_DIGEST: per-cycle flop digest
 * d_t = sum_w rotl64(zext64(Qw), w mod 64) * (2w+1) mod 2^64 over the external
 * flop words of Q(t+1); uint64 [n_streams][ncycles] (host). */
int gem_read_digests(gem_sim* sim, uint64_t* dst, uint64_t ncycles);

/* RAM block contents (8192 x 32-bit words: "13 bits address and 32 bits data",
 * P:93) of one stream, host buffers of 8192 words.  gem_write_ram preloads a
 * block before the next step (U10: otherwise 0); the registered read data RD
 * is not changed (it holds the last read, 0 before the first cycle).
 * Synchronous.  Errors: GEM_E_INVAL (null, ram_id >= n_rams, stream >= n_streams). */
int gem_read_ram(gem_sim* sim, uint32_t ram_id, uint32_t stream, uint32_t* words8192);
int gem_write_ram(gem_sim* sim, uint32_t ram_id, uint32_t stream, const uint32_t* words8192);

/* Latency-floor microbenchmarks (measurement helper for the roofline; not part
 * of the simulation path): *layer_clk = SM clocks of a minimal boomerang layer
 * (one dependent gathered load per thread, levels 1-13, write-out, block
 * barrier) on one CTA; *barrier_clk = SM clocks of one grid barrier round trip
 * among `grid` co-resident CTAs (grid <= 1024).  Allocates and frees its own
 * device memory on `device`. */
int gem_bench_floor(int device, uint32_t grid, uint32_t iters, double* layer_clk, double* barrier_clk);
/* *step_clk = SM clocks of a minimal word-mode step (GEM_F_NO_WORDS off, blobs
 * mapped with words=1): block barrier, two operand loads per thread, AND with
 * inversions, result store, on one CTA -- the per-step term of word mode's
 * latency floor.  Measurement helper, not part of the simulation path. */
int gem_bench_floor_step(int device, uint32_t iters, double* step_clk);

/* Device time (CUDA events on the launch stream) of the last gem_step kernel. */
int gem_last_step_ms(gem_sim* sim, float* ms);

/* Needs GEM_F_PROFILE: per-cycle, per-CTA SM clock64 stamps of the last step,
 * uint64 [n_cycles][grid][GEM_PROF_SLOTS = 16]: 0 cycle start, 1 input ports
 * read (after the barrier), 2 layers done, 3 endpoints+RAM committed (first
 * work item), 4 stage-0 items done, 5 after the last grid barrier, 6 = layer
 * count of the first item, 7 program chunk 0 ready, 8 input-port loads stored,
 * 9 layer-0 records loaded (before the barrier), 10 = partition id of the
 * last work item; 11-15 unused.
 * Call with dst = NULL to query n_cycles / grid. */
#define GEM_PROF_SLOTS 16
int gem_read_profile(gem_sim* sim, uint64_t* dst, uint32_t* n_cycles, uint32_t* grid);

/* Needs GEM_F_ACTIVITY: partition-cycles evaluated and skipped since load
 * (summed over CTAs eligible for pruning; ineligible CTAs are not counted). */
int gem_read_activity(gem_sim* sim, uint64_t* evaluated, uint64_t* skipped);

/* ---- Single-design multi-GPU (§V P:247 lists
 * multi-GPU as future work, so the protocol is this library's).
 * Every rank loads the same blob with the same n_streams and cfg.dist_world,
 * its own cfg.dist_rank.  A rank evaluates the partitions it owns; at each
 * endpoint commit the kernel stores the flop (Q), RAM-read (RD),
 * cut and PO words into its own buffers AND into every peer's (peer memory
 * over NVLink / PCIe, or the same device), then meets the other ranks at a
 * cross-device barrier at every stage boundary, plus once at the start of
 * each launch: every CTA of every rank stores its arrival epoch into its slot
 * of every rank's flag array (after a system-scope fence) and polls the
 * slots of its own array.  So Q, RD, cut and PO words are replicated on every rank (gem_read_*
 * of states, traces and outputs works on any rank); RAM contents (gem_read_ram
 * / gem_write_ram) live only on the rank that owns the RAM's partition.
 * Every rank must call gem_set_inputs with the same stimuli and gem_step with
 * the same cycle counts, concurrently (each call waits for the others in the
 * kernel; a rank that never comes trips the 10 s barrier watchdog). */
#define GEM_DIST_MAX 8
#define GEM_DIST_IPC_BYTES 328   /* 5 cudaIpcMemHandle_t + grid + reserved */
typedef struct {
  void* q;      /* device pointers (as seen by the connecting process) of one */
  void* rd;     /* rank's replicated buffers and its barrier flags            */
  void* cut;
  void* po;
  void* flags;
  uint32_t grid;       /* CTAs of that rank's launches (its barrier slots) */
  uint32_t reserved;
} gem_dist_buffers;

/* Host-only (no CUDA call): owner rank of each partition for a world of
 * `world` ranks, written to owner[n_parts]: per stage, partitions in
 * decreasing mapper cost to the least-loaded rank (ties: less work in the
 * earlier stages, then the lower rank).
 * Deterministic, so every rank computes the same split.  Errors: GEM_E_INVAL,
 * GEM_E_FORMAT (as gem_load_program). */
int gem_dist_owner(const void* blob, size_t nbytes, uint32_t world, uint32_t* owner);

/* This rank's buffers for its peers.  Fixes the output capacity at
 * max_cycles (a later gem_step of more cycles per call is GEM_E_INVAL) and
 * allocates the zeroed barrier flags.  Errors: GEM_E_INVAL (not a dist handle,
 * max_cycles 0 or > 2^32-16), GEM_E_NOMEM, GEM_E_CUDA. */
int gem_dist_export(gem_sim* sim, uint64_t max_cycles, gem_dist_buffers* out);
/* The exported buffers as CUDA IPC handles (GEM_DIST_IPC_BYTES host bytes)
 * for a peer in another process; call after gem_dist_export. */
int gem_dist_ipc_handles(gem_sim* sim, void* out);
/* Maps a peer process's handles into this process (closed by gem_free);
 * *out receives pointers for gem_dist_connect. */
int gem_dist_ipc_open(gem_sim* sim, const void* handles, gem_dist_buffers* out);
/* Peer buffers of every rank (peers[dist_world], peers[dist_rank] ignored;
 * same-process pointers on another device get peer access enabled).
 * Errors: GEM_E_INVAL (not exported, null entry), GEM_E_CUDA. */
int gem_dist_connect(gem_sim* sim, const gem_dist_buffers* peers);

void gem_free(gem_sim* sim);
const char* gem_last_error(void);

#ifdef __cplusplus
}
#endif
#endif /* GEM_H */
