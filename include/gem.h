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

typedef struct gem_sim gem_sim; /* opaque, owned by the library */

typedef struct {
  int device;           /* CUDA device ordinal                                     */
  uint32_t n_streams;   /* independent stimulus streams over the same design (>=1) */
  void* cuda_stream;    /* cudaStream_t to launch on, or NULL for a private stream */
  uint32_t flags;       /* GEM_F_*                                                 */
  uint32_t grid_limit;  /* 0 = auto (co-resident persistent grid); else max CTAs   */
} gem_config;

typedef struct {
  uint32_t n_pi, n_po, n_flops, n_rams, n_parts, n_stages, max_layers, total_layers;
  uint32_t pi_words, po_words, q_words;   /* external word counts per cycle/stream */
  uint32_t grid, blocks_per_sm, smem_bytes, n_streams;
  uint32_t resident;     /* CTAs whose programs all live in their shared memory */
  uint32_t ring_slots;   /* else: TMA ring depth used to stream program chunks */
  uint32_t group;        /* streams per work item (program chunks reused across them) */
  uint32_t lanes;        /* 1 = stream-sliced lane mode (32 streams per lane word)  */
  uint64_t n_and;                          /* live 2-input ANDs (gate evals/cycle) */
  uint64_t n_and_mapped;                   /* with RepCut replication              */
  uint64_t program_bytes;
  uint64_t cycle;                          /* cycles simulated so far              */
} gem_info;

/* Load a .gemb program blob (mapper output), allocate device state for
 * cfg->n_streams streams; flops start at their AIGER init values, RAMs at 0
 * (readings U5, U10).  blob: host memory, nbytes bytes; copied. */
int gem_load_program(const void* blob, size_t nbytes, const gem_config* cfg, gem_sim** out);

int gem_info_get(const gem_sim* sim, gem_info* out);

/* Queue ncycles of primary-input vectors for every stream:
 * pi_words = uint32 [n_streams][ncycles][pi_words] (host, or device if
 * src_on_device).  Replaces any inputs not yet consumed. */
int gem_set_inputs(gem_sim* sim, const uint32_t* pi_words, uint64_t ncycles, int src_on_device);

/* Simulate ncycles cycles (consumes ncycles queued input vectors) with one
 * persistent cooperative kernel launch.  After return, state = Q[t0+ncycles]. */
int gem_step(gem_sim* sim, uint64_t ncycles);

/* PO[t0 .. t0+ncycles-1] of the last gem_step, sampled before each clock edge
 * (reading U11): uint32 [n_streams][ncycles][po_words]. */
int gem_read_outputs(gem_sim* sim, uint32_t* po_words, uint64_t ncycles, int dst_on_device);

/* Current flop vector: uint32 [n_streams][q_words], AIGER latch order. */
int gem_read_state(gem_sim* sim, uint32_t* flop_words, int dst_on_device);
int gem_write_state(gem_sim* sim, const uint32_t* flop_words, int src_on_device);

/* Needs GEM_F_TRACE_STATE: Q(t+1) for every cycle of the last step,
 * uint32 [n_streams][ncycles][q_words] (host). */
int gem_read_state_trace(gem_sim* sim, uint32_t* dst, uint64_t ncycles);

/* Needs GEM_F_DIGEST: d_t = sum_w rotl64(zext64(Qw), w mod 64) * (2w+1) mod 2^64
 * over the external flop words of Q(t+1); uint64 [n_streams][ncycles] (host). */
int gem_read_digests(gem_sim* sim, uint64_t* dst, uint64_t ncycles);

/* RAM block contents (8192 x 32-bit words) of one stream (host buffers). */
int gem_read_ram(gem_sim* sim, uint32_t ram_id, uint32_t stream, uint32_t* words8192);
int gem_write_ram(gem_sim* sim, uint32_t ram_id, uint32_t stream, const uint32_t* words8192);

/* Latency-floor microbenchmarks (measurement helper for the roofline; not part
 * of the simulation path): *layer_clk = SM clocks of a minimal boomerang layer
 * (one dependent gathered load per thread, levels 1-13, write-out, block
 * barrier) on one CTA; *barrier_clk = SM clocks of one grid barrier round trip
 * among `grid` co-resident CTAs (grid <= 1024).  Allocates and frees its own
 * device memory on `device`. */
int gem_bench_floor(int device, uint32_t grid, uint32_t iters, double* layer_clk, double* barrier_clk);

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

void gem_free(gem_sim* sim);
const char* gem_last_error(void);

#ifdef __cplusplus
}
#endif
#endif /* GEM_H */
