// gem_runtime.cu -- libgem: C ABI (include/gem.h) + the sm_100a GEM VLIW
// interpreter kernel.
//
// Per simulated cycle:
//   for each stage s:
//     every CTA runs the partitions (x streams) of stage s assigned to it:
//       a2  global read: copy the partition's input-port words (PI[t], Q_cur,
//           RD_cur, stage-cut words) into the shared-memory state S
//       a3  per layer: gather the used leaves of each thread's 32-bit leaf
//           word from S (bit permutation)
//       a4  boomerang fold: levels 1-5 in-thread, levels 6-10 in-warp after a
//           ballot, levels 11-13 across warps  (P:85, P:81 word parallelism)
//       a5  write-outs of packed slot words into free state words
//       a6  endpoint commit: warp ballot-gathers of endpoint bits into owned
//           global words Q_next / PO[t] / CUT / RAM-port staging
//       a7  RAM blocks owned by the partition: read-first, then per-bit write
//     a8  grid-wide barrier (own acquire/release counter barrier on a
//         cooperative, co-resident persistent grid)
// No tensor cores (not a contraction), no library calls, no CPU fallback.
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <string>
#include <vector>

#include "gem.h"
#include "gem_isa.h"

namespace {

thread_local std::string g_err;

// streams (packed) or 32-stream groups (lanes) per work item: each uses its own
// named barrier 1..15 for the top levels (barrier 0 = __syncthreads)
#define GEM_MAX_GROUP 15u

struct KParams {
  const uint32_t* __restrict__ prog;
  const uint32_t* __restrict__ parts;       // part table [n_parts][4]
  const uint32_t* __restrict__ stage_list;  // [n_stages+1] prefix, then part ids
  const uint32_t* __restrict__ pi;          // [stream][in_cap][pi_words]
  uint32_t* po;                             // [stream][out_cap][po_words_int]
  uint32_t* q;                              // [2][stream][q_words_int]
  uint32_t* rd;                             // [2][stream][n_rams]
  uint32_t* cut;                            // [stream][cut_words]
  uint32_t* mem;                            // [stream][n_rams][8192]
  uint32_t* q_trace;                        // [stream][out_cap][q_ext_words]
  unsigned long long* digest;               // [stream][out_cap]
  const uint32_t* __restrict__ q_int_of_ext;  // [n_flops] internal bit
  unsigned long long* bar;                  // grid barrier: per-CTA arrival flags
  uint32_t* err;                            // mapped pinned host words {code, cta, flag, epoch}
  uint64_t t0;
  uint32_t ncycles, in_base, in_cap, out_cap;
  uint32_t n_stages, n_streams, state_words;
  uint32_t pi_words, po_words, q_words, cut_words, n_rams, n_flops, q_ext_words;
  uint32_t flags;
  uint32_t area_words, slot_words, ring_slots, allow_resident;
  unsigned long long* prof;   // GEM_F_PROFILE: [prof_cycles][grid][GEM_PROF_SLOTS] clock64 stamps
  uint32_t prof_cycles;
  uint32_t group;                        // streams per work item (stream states in smem)
  // lane mode
  const uint32_t* __restrict__ lprog;    // lane programs
  const uint32_t* __restrict__ pi_lane;  // [in_cap][pi_words*32][n_groups]
  uint32_t* po_lane;                     // [out_cap][po_words*32][n_groups]
  uint32_t n_groups, ramp_words;
  const uint32_t* __restrict__ wl_off;   // [n_stages][grid+1] CSR offsets into wl_items
  const uint2* __restrict__ wl_items;    // {partition, stream} per work item
  // GEM_F_ACTIVITY (row f3): per-CTA copy of the last input-port words
  // (act_words >= max n_gread) and {evaluated, skipped} partition-cycle counters
  unsigned long long* act_cnt;
  uint32_t act_words;
  // single-CTA launches (LOC kernels): the flop / RAM-read words live in shared
  // memory across cycles, [2][loc_words] with loc_words = q_words + n_rams
  uint32_t loc_words;
  float l2_frac;           // > 0: streamed program chunks keep this fraction evict_last in L2
  // lane mode, one stage: dynamic work distribution.  Units {partition, first
  // stream, items, 0} in LPT order; CTA b starts every cycle with unit b and
  // then takes tickets from dyn_ctr[cycle & 1] (+ grid).
  const uint4* __restrict__ dyn_units;
  uint32_t n_units;
  uint32_t* dyn_ctr;
  // single-design multi-GPU (DIST kernels, include/gem.h gem_dist_*): committed
  // Q / RD / cut / PO words are also stored into every peer's buffers, and the
  // grid barrier meets the peers' through system-scope flags (epochs continue
  // across launches: dist_epoch0 = barriers of earlier launches)
  uint32_t dist_world, dist_rank;
  unsigned long long dist_epoch0;
  unsigned long long* dist_flags;              // this rank's flags [world][GEM_BAR_MAX_CTAS] (x stride)
  unsigned long long* peer_flags[GEM_DIST_MAX];  // every rank's flags (this rank's = dist_flags)
  uint32_t dist_grid[GEM_DIST_MAX];            // CTAs of each rank's launch
  uint32_t dist_slots;                         // sum of dist_grid
  uint32_t* peer_q[GEM_DIST_MAX];
  uint32_t* peer_rd[GEM_DIST_MAX];
  uint32_t* peer_cut[GEM_DIST_MAX];
  uint32_t* peer_po[GEM_DIST_MAX];
};
#define PROF(slot_)                                                                          \
  do {                                                                                       \
    if (prof_on && threadIdx.x == 0)                                                         \
      kp.prof[((size_t)c * gridDim.x + blockIdx.x) * GEM_PROF_SLOTS + (slot_)] = (unsigned long long)clock64(); \
  } while (0)

__device__ __forceinline__ unsigned long long ld_acquire_u64(const unsigned long long* p) {
  unsigned long long v;
  asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}

__device__ __forceinline__ uint64_t globaltimer_ns() {
  uint64_t t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}

// Grid-wide barrier on per-CTA arrival flags (one 128-byte line each, reset to
// 0 before each launch).  Arrive: bar.sync, then thread 0 stores the barrier
// epoch with st.release.gpu (cumulative over the CTA's writes ordered before it
// by the bar.sync).  Wait: thread f polls CTA f's flag with ld.acquire.gpu (all
// flags in parallel, no single contended counter), then bar.sync.  A 10 s spin
// limit turns a deadlock (e.g. broken co-residency) into a trapped kernel; the
// watchdog first sets KParams::err (mapped pinned host memory), which the host
// reads after the failed synchronisation so the error names the barrier (the
// context itself is lost).  The watchdog is kept to one atomic + trap: a richer
// report in this loop (CAS + stores + fence) slowed C3's cycle by 1-5%.
// (Measured alternatives: relaxed polling + one fence, a
// two-phase gather by CTA 0, a single red.release counter: all slower.)
#define GEM_BAR_STRIDE 16   /* u64 words between flags (128 bytes) */
#define GEM_BAR_MAX_CTAS 1024
#define GEM_WATCHDOG_NS 10000000000ull
#define GEM_ERR_BARRIER 2u
__device__ __forceinline__ void st_release_u64(unsigned long long* p, unsigned long long v) {
  asm volatile("st.release.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ void spin_check(uint32_t& spins, uint64_t& start, const KParams& kp, uint32_t flag,
                                           unsigned long long epoch) {
  if (++spins == 4096) start = globaltimer_ns();
  if (spins > 4096 && (spins & 4095) == 0 && globaltimer_ns() - start > GEM_WATCHDOG_NS) {
    atomicExch(kp.err, GEM_ERR_BARRIER);
    asm volatile("trap;");
  }
}
__device__ __forceinline__ unsigned long long ld_acquire_sys_u64(const unsigned long long* p) {
  unsigned long long v;
  asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
// DIST: a committed word to every peer's copy of the same buffer (same offset)
__device__ __forceinline__ void dist_put(const KParams& kp, uint32_t* const* peers, size_t off, uint32_t v) {
  for (uint32_t r = 0; r < kp.dist_world; r++)
    if (r != kp.dist_rank) __stcg(peers[r] + off, v);
}
template <bool DIST = false>
__device__ __forceinline__ void grid_sync(const KParams& kp, unsigned long long& epoch) {
  if (DIST) {
    // Cross-device barrier, flat like the single-device one: after bar.sync,
    // thread 0 makes the CTA's stores (local and peer) visible at system scope
    // (fence.acq_rel.sys, cumulative over the CTA's writes ordered by the
    // bar.sync) and stores the epoch into this CTA's slot of EVERY rank's flag
    // array (slot rank * GEM_BAR_MAX_CTAS + cta; its own included); then
    // thread f polls slot f of its own array (ld.acquire.sys; all ranks' CTAs).
    // Epochs continue across launches (the flags are never reset).
    // Measured on one B200 with in-process ranks (scripts/split_bench.py, C3,
    // 2 ranks): 14.8 us per cycle vs 10.5 single-rank; the system-scope fence
    // is 3.4 us of it (a gpu-scope one, not valid across devices: 11.4 us);
    // a fence in every committing thread, or a two-level gather through CTA 0,
    // was slower (18-22 us, 19.5 us).
    __syncthreads();
    epoch++;
    const unsigned long long de = kp.dist_epoch0 + epoch;
    if (threadIdx.x == 0) {
      asm volatile("fence.acq_rel.sys;" ::: "memory");
      const size_t slot = ((size_t)kp.dist_rank * GEM_BAR_MAX_CTAS + blockIdx.x) * GEM_BAR_STRIDE;
      for (uint32_t r = 0; r < kp.dist_world; r++)
        asm volatile("st.relaxed.sys.global.u64 [%0], %1;" ::"l"(kp.peer_flags[r] + slot), "l"(de) : "memory");
    }
    for (uint32_t f = threadIdx.x; f < kp.dist_slots; f += blockDim.x) {
      uint32_t r = 0, b = f;
      while (b >= kp.dist_grid[r]) b -= kp.dist_grid[r++];
      const unsigned long long* fl = kp.dist_flags + ((size_t)r * GEM_BAR_MAX_CTAS + b) * GEM_BAR_STRIDE;
      uint32_t spins = 0;
      uint64_t start = 0;
      while (ld_acquire_sys_u64(fl) < de) spin_check(spins, start, kp, f, de);
    }
    __syncthreads();
    return;
  }
  __syncthreads();
  if (gridDim.x > 1) {
    epoch++;
    if (threadIdx.x == 0) st_release_u64(kp.bar + (size_t)blockIdx.x * GEM_BAR_STRIDE, epoch);
    for (uint32_t f = threadIdx.x; f < gridDim.x; f += blockDim.x) {
      uint32_t spins = 0;
      uint64_t start = 0;
      while (ld_acquire_u64(kp.bar + (size_t)f * GEM_BAR_STRIDE) < epoch) spin_check(spins, start, kp, f, epoch);
    }
    __syncthreads();
  }
}

// Levels 1-5 (or 6-10) of the boomerang fold on one 32-bit word.  The
// constants stay in their packed slot positions (gem_isa.h: L1 bits [0,16),
// L2 [16,24), L3 [24,28), L4 [28,30), L5 [30]); the data of level k is shifted
// into level k's field instead (2 shifts + 2 LOP3 per level), and the packed
// result is assembled with bit-selects.  Bits outside each level's field are
// don't-care.
__device__ __forceinline__ uint32_t bsel(uint32_t a, uint32_t b, uint32_t m) { return (a & ~m) | (b & m); }
__device__ __forceinline__ uint32_t fold5(uint32_t v, uint32_t xa, uint32_t xb, uint32_t ob) {
  const uint32_t r1 = (v ^ xa) & (((v >> 16) ^ xb) | ob);                  // [0,16): A=v[q], B=v[q+16]
  const uint32_t r2 = ((r1 << 16) ^ xa) & (((r1 << 8) ^ xb) | ob);         // [16,24): A=r1[q], B=r1[q+8]
  const uint32_t r3 = ((r2 << 8) ^ xa) & (((r2 << 4) ^ xb) | ob);          // [24,28): A=r2[16+q], B=r2[20+q]
  const uint32_t r4 = ((r3 << 4) ^ xa) & (((r3 << 2) ^ xb) | ob);          // [28,30)
  const uint32_t r5 = ((r4 << 2) ^ xa) & (((r4 << 1) ^ xb) | ob);          // [30]
  return bsel(bsel(bsel(bsel(r1, r2, 0x00FF0000u), r3, 0x0F000000u), r4, 0x30000000u), r5, 0xC0000000u) &
         0x7FFFFFFFu;
}

// Levels 11-13 on the 8 warp bits.
__device__ __forceinline__ uint32_t fold3(uint32_t v, uint32_t xa, uint32_t xb, uint32_t ob) {
  uint32_t r1 = (v ^ xa) & (((v >> 4) ^ xb) | ob);
  uint32_t r2 = (r1 ^ (xa >> 4)) & (((r1 >> 2) ^ (xb >> 4)) | (ob >> 4));
  uint32_t r3 = (r2 ^ (xa >> 6)) & (((r2 >> 1) ^ (xb >> 6)) | (ob >> 6));
  return (r1 & 0xFu) | ((r2 & 3u) << 4) | ((r3 & 1u) << 6);
}

__device__ __forceinline__ uint32_t rd_global(const uint32_t* p) { return __ldcg(p); }

// ---------------------------------------------------------------- TMA / mbarrier
__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return (uint32_t)__cvta_generic_to_shared(p);
}
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t* bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes)
               : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
  // (no watchdog here: even an out-of-line slow path cost ~70 clk per C3
  // layer; a grid-barrier stall still traps after 10 s)
  uint32_t done = 0;
  while (!done) {
    asm volatile(
        "{\n .reg .pred p;\n mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n selp.u32 %0, 1, 0, p;\n}\n"
        : "=r"(done)
        : "r"(smem_u32(bar)), "r"(parity)
        : "memory");
  }
}
// 1-D bulk copy global -> shared (TMA engine), completion signalled on `bar`.
// bytes must be a multiple of 16 and both addresses 16-byte aligned.
__device__ __forceinline__ void tma_load_1d(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
          smem_u32(dst)),
      "l"(src), "r"(bytes), "r"(smem_u32(bar))
      : "memory");
}
// The same copy with an L2 cache-eviction policy (createpolicy): programs larger
// than the L2 stream every cycle; keeping a fraction of their lines evict_last
// (the rest evict_first) lets that fraction stay L2-resident across cycles.
__device__ __forceinline__ void tma_load_1d_hint(void* dst, const void* src, uint32_t bytes, uint64_t* bar,
                                                 uint64_t pol) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1], %2, [%3], %4;" ::"r"(
          smem_u32(dst)),
      "l"(src), "r"(bytes), "r"(smem_u32(bar)), "l"(pol)
      : "memory");
}
__device__ __forceinline__ uint64_t l2_policy(float frac) {
  uint64_t pol;
  asm volatile("createpolicy.fractional.L2::evict_last.L2::evict_first.b64 %0, %1;" : "=l"(pol) : "f"(frac));
  return pol;
}
__device__ __forceinline__ uint64_t l2_policy_unchanged() {
  uint64_t pol;
  asm volatile("createpolicy.fractional.L2::evict_unchanged.b64 %0, 1.0;" : "=l"(pol));
  return pol;
}
__device__ __forceinline__ void fence_mbar_init() {
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}

#define GEM_RING_MAX 8
#define GEM_MAX_RESIDENT 16
#define GEM_WL_MAX_STAGES 8
#define GEM_WL_CACHE 64                              // work items cached in smem per CTA
#define GEM_WL_CACHE_WORDS (32 + 2 * GEM_WL_CACHE)

// Shared-memory program source: either every program of this CTA resident
// (copied once per launch) or a ring of R slots fed chunk by chunk by TMA.
struct ProgSrc {
  uint64_t* mbar;        // [GEM_RING_MAX + 1]; last one = residency barrier
  uint32_t* area;        // resident programs or ring slots
  uint32_t* ctab;        // chunk table copy (streamed mode)
  uint32_t slot_words, R;
  uint32_t seq_issue, seq_wait, seq_free;   // chunk sequence numbers (uniform across the CTA)
  bool resident;
  // pinned prefix (single-partition CTAs whose program does not fit): chunks
  // [0, pin_chunks) stay in `pin` for the launch, the rest stream through the
  // ring placed after them; pro_chunk/pro_off = next chunk after the prologue
  uint32_t pin_chunks, pin_off, pro_chunk, pro_off;
  const uint32_t* pin;
  uint64_t l2pol;          // L2 policy of streamed chunks (KParams::l2_frac)
  uint32_t n_res;
  const uint32_t* res_p;   // smem [GEM_MAX_RESIDENT] partition ids
  const uint32_t* res_off; // smem [GEM_MAX_RESIDENT] word offsets into area
};

// ring depth R is a power of two (2, 4 or 8): slot = seq & (R-1), phase = (seq / R) & 1
__device__ __forceinline__ uint32_t* ring_slot(const ProgSrc& ps, uint32_t seq) {
  return ps.area + (seq & (ps.R - 1)) * ps.slot_words;
}
// All threads call this (uniformly); thread 0 issues the copy.
__device__ __forceinline__ void ring_issue(ProgSrc& ps, const uint32_t* g, uint32_t words) {
  const uint32_t seq = ps.seq_issue++;
  if (threadIdx.x == 0) {
    uint64_t* bar = ps.mbar + (seq & (ps.R - 1));
    mbar_expect_tx(bar, words * 4);
    tma_load_1d_hint(ring_slot(ps, seq), g, words * 4, bar, ps.l2pol);
  }
}
__device__ __forceinline__ const uint32_t* ring_wait(ProgSrc& ps) {
  const uint32_t seq = ps.seq_wait++;
  mbar_wait(ps.mbar + (seq & (ps.R - 1)), (seq >> (__ffs(ps.R) - 1)) & 1u);   // phase = (seq / R) & 1
  return ring_slot(ps, seq);
}

// Prologue of a work item in streamed mode: its first min(R, 3, n_chunks)
// chunks, sized from the partition table (issued before the item starts,
// e.g. while the CTA waits at the grid barrier).
__device__ __forceinline__ uint32_t prologue_count(const KParams& kp, const ProgSrc& ps, uint32_t p) {
  const uint32_t nch = __ldg(kp.parts + p * GP_WORDS + GP_N_LAYERS) + 2;
  return min(min(ps.R, 3u), nch);
}
__device__ __forceinline__ void issue_prologue(const KParams& kp, ProgSrc& ps, uint32_t p) {
  const uint32_t* g = kp.prog + __ldg(kp.parts + p * GP_WORDS + GP_PROG_OFF);
  const uint32_t k = prologue_count(kp, ps, p);
  const uint32_t sz[3] = {__ldg(kp.parts + p * GP_WORDS + GP_CHUNK0), __ldg(kp.parts + p * GP_WORDS + GP_CHUNK1),
                          __ldg(kp.parts + p * GP_WORDS + GP_CHUNK2)};
  uint32_t off = 0;
  for (uint32_t i = 0; i < k; i++) {
    ring_issue(ps, g + off, sz[i]);
    off += sz[i];
  }
}

// Prologue in pinned-prefix mode: the first streamed chunks of partition p
// (sizes from the pinned chunk table); records where refilling resumes.
__device__ __forceinline__ void issue_prologue_pinned(const KParams& kp, ProgSrc& ps, uint32_t p) {
  const uint32_t* g = kp.prog + __ldg(kp.parts + p * GP_WORDS + GP_PROG_OFF);
  const uint32_t* ct = ps.pin + ps.pin[PH_OFF_CHUNKS];
  const uint32_t nch = ps.pin[PH_N_CHUNKS];
  uint32_t k = ps.pin_chunks, off = ps.pin_off;
  while (k < nch && k < ps.pin_chunks + ps.R) {
    ring_issue(ps, g + off, ct[k]);
    off += ct[k];
    k++;
  }
  ps.pro_chunk = k;
  ps.pro_off = off;
}

// Explicit shared-window accesses (32-bit addresses): avoids generic->shared
// conversions in the hot loops.
__device__ __forceinline__ uint32_t lds(uint32_t addr) {
  uint32_t v;
  asm volatile("ld.shared.u32 %0, [%1];" : "=r"(v) : "r"(addr));
  return v;
}
__device__ __forceinline__ void sts(uint32_t addr, uint32_t v) {
  asm volatile("st.shared.u32 [%0], %1;" ::"r"(addr), "r"(v) : "memory");
}

// Gather of one leaf entry: rotate the source state word so bit b lands on
// leaf position p (gem_isa.h).  S sits at the start of dynamic shared memory,
// so the entry's byte-offset field plus the window base addresses it.
// Dynamic shared memory of both kernels; the partition state S is at offset 0.
extern __shared__ __align__(16) uint32_t g_smem[];

// Gather loads are plain C++ loads from the shared-memory state (the compiler
// keeps the per-stream base in a uniform register: LDS [R + UR], no per-leaf add).
__device__ __forceinline__ uint32_t ldsb(const uint32_t* S, uint32_t byteoff) {
  return *reinterpret_cast<const uint32_t*>(reinterpret_cast<const char*>(S) + byteoff);
}
// Single-stream fast path: the state sits at the start of dynamic shared
// memory, shared-window address GEM_S0_ADDR (checked at kernel start), so the
// base is an LDS immediate and a leaf's address is just its byte offset.
#define GEM_S0_ADDR 1024
template <bool kS0>
__device__ __forceinline__ uint32_t ldst(const uint32_t* S, uint32_t byteoff) {
  if (kS0) {
    uint32_t v;
    asm volatile("ld.shared.u32 %0, [%1+1024];" : "=r"(v) : "r"(byteoff));
    return v;
  }
  return ldsb(S, byteoff);
}
// load address = entry >> 16 (byte offset), rotation = low 5 bits (gem_isa.h)
template <bool kS0 = false>
__device__ __forceinline__ uint32_t leaf_rot(const uint32_t* S, uint32_t e) {
  const uint32_t s = ldst<kS0>(S, e >> 16);
  return __funnelshift_l(s, s, e);   // rotl(s, e & 31)
}
// SPARSE entry: position mask rotl(1, e >> 8) (low 5 bits = leaf position)
__device__ __forceinline__ uint32_t leaf_mask(uint32_t e) { return __funnelshift_l(1u, 1u, e >> 8); }
template <int N4, bool kS0>
__device__ __forceinline__ uint32_t gather_sparse(const uint32_t* S, const uint4* e) {
  // four independent accumulators keep the OR chain short
  uint32_t v0 = 0, v1 = 0, v2 = 0, v3 = 0;
#pragma unroll
  for (int g = 0; g < N4; g++) {
    v0 |= leaf_rot<kS0>(S, e[g].x) & leaf_mask(e[g].x);
    v1 |= leaf_rot<kS0>(S, e[g].y) & leaf_mask(e[g].y);
    v2 |= leaf_rot<kS0>(S, e[g].z) & leaf_mask(e[g].z);
    v3 |= leaf_rot<kS0>(S, e[g].w) & leaf_mask(e[g].w);
  }
  return (v0 | v1) | (v2 | v3);
}

// Per-thread registers of one layer record: everything that does not depend
// on the state, so it can be loaded before the barrier of the previous layer.
struct LayerRegs {
  uint4 e[8];
  uint4 lc, wc;
  uint32_t cls, flags, topc, topwo;
  uint32_t ndir;   // this warp's entry of the next layer's record directory
};

// uint4 leaf groups per lane of a record class (gem_isa.h GEM_DC_*)
__device__ __forceinline__ uint32_t dc_n4(uint32_t cls) {
  return cls <= 8u ? cls : (cls == GEM_DC_DENSE16 ? 4u : 8u);
}

// `dir` = this warp's directory entry for layer L (from the previous layer's
// header, or chunk 0 for layer 0): the record address is known up front, so
// every load below is independent and issues back to back.
__device__ __forceinline__ void load_layer(const uint32_t* L, uint32_t dir, LayerRegs& R) {
  const uint32_t lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const uint4 lh0 = *reinterpret_cast<const uint4*>(L);
  const uint32_t nd = L[LH_NEXTDIR + (warp >> 1)];
  R.flags = lh0.y;
  R.topc = lh0.z;
  R.topwo = lh0.w;
  R.ndir = (nd >> (16u * (warp & 1u))) & 0xFFFFu;
  R.cls = dir >> 12;
  if (R.cls) {
    const uint32_t* rec = L + 4u * (dir & 0xFFFu);
    R.wc = *reinterpret_cast<const uint4*>(rec);
    R.lc = *(reinterpret_cast<const uint4*>(rec + GEM_WREC_HDR) + lane);
    const uint4* lv = reinterpret_cast<const uint4*>(rec + GEM_WREC_HDR + 128) + lane;
    const uint32_t n4 = dc_n4(R.cls);
#pragma unroll
    for (uint32_t g = 0; g < 8; g++) R.e[g] = g < n4 ? lv[g * 32] : make_uint4(0u, 0u, 0u, 0u);
  }
}
// directory entry of this warp for layer 0 (chunk 0)
__device__ __forceinline__ uint32_t dir0_entry(const uint32_t* C0, uint32_t off_dir0) {
  const uint32_t warp = threadIdx.x >> 5;
  return (C0[off_dir0 + (warp >> 1)] >> (16u * (warp & 1u))) & 0xFFFFu;
}

// Rows a3-a5 of one layer with pre-loaded records: gather (bit permutation),
// 13-level boomerang fold, write-outs.  No trailing barrier.
template <bool kS0>
__device__ __forceinline__ void exec_layer(const LayerRegs& R, uint32_t s_base, const uint32_t* Sj, uint32_t* topb,
                                           uint32_t bid) {
  const uint32_t lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const bool uses_top = (R.flags & GEM_LF_USES_TOP) != 0;
  if ((R.flags >> warp) & 1u) {
    uint32_t v = 0;
    const uint32_t n4 = dc_n4(R.cls);
    if (R.cls == GEM_DC_DENSE16) {
      // two 16-bit entries per u32: entry 8g+2k in the low half, 8g+2k+1 in the high half
      uint32_t acc[4] = {0u, 0u, 0u, 0u};
#pragma unroll
      for (uint32_t g = 0; g < 4; g++) {
        const uint32_t q[4] = {R.e[g].x, R.e[g].y, R.e[g].z, R.e[g].w};
#pragma unroll
        for (uint32_t k = 0; k < 4; k++) {
          const uint32_t lo = ldst<kS0>(Sj, (q[k] >> 3) & 0x1FFCu);
          const uint32_t hi = ldst<kS0>(Sj, (q[k] >> 19) & 0x1FFCu);
          acc[k] |= (__funnelshift_l(lo, lo, q[k]) & (1u << (8 * g + 2 * k))) |
                    (__funnelshift_l(hi, hi, q[k] >> 16) & (1u << (8 * g + 2 * k + 1)));
        }
      }
      v = (acc[0] | acc[1]) | (acc[2] | acc[3]);
    } else if (R.cls == GEM_DC_DENSE) {
      // entry j of the lane fills leaf position j: rotate + LOP3 with an immediate mask
#pragma unroll
      for (uint32_t g = 0; g < 8; g++) {
        v |= leaf_rot<kS0>(Sj, R.e[g].x) & (1u << (4 * g + 0));
        v |= leaf_rot<kS0>(Sj, R.e[g].y) & (1u << (4 * g + 1));
        v |= leaf_rot<kS0>(Sj, R.e[g].z) & (1u << (4 * g + 2));
        v |= leaf_rot<kS0>(Sj, R.e[g].w) & (1u << (4 * g + 3));
      }
    } else {
      switch (n4) {
        case 1: v = gather_sparse<1, kS0>(Sj, R.e); break;
        case 2: v = gather_sparse<2, kS0>(Sj, R.e); break;
        case 3: v = gather_sparse<3, kS0>(Sj, R.e); break;
        case 4: v = gather_sparse<4, kS0>(Sj, R.e); break;
        case 5: v = gather_sparse<5, kS0>(Sj, R.e); break;
        case 6: v = gather_sparse<6, kS0>(Sj, R.e); break;
        case 7: v = gather_sparse<7, kS0>(Sj, R.e); break;
        default: v = gather_sparse<8, kS0>(Sj, R.e); break;
      }
    }
    const uint32_t P = fold5(v, R.lc.x, R.lc.y, R.lc.z);
    if (R.lc.w) sts(s_base + 4 * R.lc.w, P);
    const uint32_t u = __ballot_sync(0xFFFFFFFFu, (P >> 30) & 1u);
    const uint32_t Pw = fold5(u, R.wc.x, R.wc.y, R.wc.z);
    if (lane == 0) {
      if (R.wc.w) sts(s_base + 4 * R.wc.w, Pw);
      if (uses_top) topb[warp] = (Pw >> 30) & 1u;
    }
  } else if (uses_top && lane == 0) {
    topb[warp] = 0u;
  }
  // levels 11-13: warps 1-7 arrive (non-blocking) on named barrier `bid`
  // after publishing their level-10 bit; warp 0 folds later (top_layer).
  if (uses_top && warp != 0) asm volatile("bar.arrive %0, %1;" ::"r"(bid), "r"(GEM_THREADS) : "memory");
}

// Levels 11-13 of a layer (warp 0 only): wait on named barrier `bid` for the
// 8 level-10 bits, fold them and write the top word.  Called after warp 0 has
// loaded the next layer's records; the layer's closing __syncthreads orders
// the write-out before the next gather.  (Measured alternatives: a smem
// atomic "last warp folds" costs ~2x; every warp folding redundantly after the
// barrier costs ~+170 clocks per layer.)
__device__ __forceinline__ void top_layer(uint32_t topc, uint32_t topwo, uint32_t s_base, const uint32_t* topb,
                                          uint32_t bid) {
  asm volatile("bar.sync %0, %1;" ::"r"(bid), "r"(GEM_THREADS) : "memory");
  if ((threadIdx.x & 31) == 0) {
    uint32_t t8 = 0;
#pragma unroll
    for (uint32_t w = 0; w < GEM_WARPS; w++) t8 |= topb[w] << w;
    sts(s_base + 4 * topwo, fold3(t8, topc & 0xFFu, (topc >> 8) & 0xFFu, (topc >> 16) & 0xFFu));
  }
}

// One work item = one partition for a group of `nst` streams (states S_j =
// S + j*state_words) in one cycle; every program chunk is loaded once and
// applied to all streams of the group.  In streamed mode the caller has
// already issued the item's prologue chunks.
// act != nullptr (GEM_F_ACTIVITY, CTA runs this one partition of one stream):
// the input-port words are compared with the previous cycle's copy in `act`
// before they enter S; if none changed (and !act_first) the layers are skipped
// -- S still holds the previous evaluation of the same inputs, so the endpoint
// commit below re-stores the same words (row f3).
// ACT = false compiles to the plain path (no activity code in the hot loop).
// LOC (single-CTA launch of one partition and one stream, gem_step_kernel<.., true>):
// every flop and RAM-read word this partition reads was written by itself in
// the previous cycle, so they come from the shared-memory copy `loc` (no L2
// round trip), and the PI words of cycle c+1 are loaded into `pv` during
// cycle c (their latency hides behind the layers).
template <bool ACT, bool LOC, bool DIST>
__device__ void run_partition(const KParams& kp, ProgSrc& ps, uint32_t* S, uint32_t* ramp, uint32_t* topb,
                              uint32_t p, uint32_t st0, uint32_t nst, uint32_t c, uint32_t cur, uint32_t nxt,
                              bool prof_on, uint32_t* act = nullptr, bool act_first = true,
                              uint32_t* loc = nullptr, uint32_t (*pv)[4] = nullptr) {
  const uint32_t tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const uint32_t SW = kp.state_words;
  const uint32_t s_base = smem_u32(S);
  const uint32_t* gprog = kp.prog + __ldg(kp.parts + p * GP_WORDS + GP_PROG_OFF);
  const uint32_t* C0;
  const uint32_t* ctab;    // chunk sizes (smem)
  uint32_t next_chunk = 0, next_off = 0;
  uint32_t n_pin = 0;      // leading chunks served from smem without the ring
  if (ps.resident) {
    uint32_t off = 0;
    for (uint32_t k = 0; k < ps.n_res; k++) if (ps.res_p[k] == p) off = ps.res_off[k];
    C0 = ps.area + off;
    ctab = C0 + C0[PH_OFF_CHUNKS];
    n_pin = ~0u;
    PROF(7);
  } else if (ps.pin_chunks) {
    C0 = ps.pin;
    ctab = C0 + C0[PH_OFF_CHUNKS];
    n_pin = ps.pin_chunks;
    next_chunk = ps.pro_chunk;
    next_off = ps.pro_off;
    PROF(7);
  } else {
    next_chunk = prologue_count(kp, ps, p);
    next_off = __ldg(kp.parts + p * GP_WORDS + GP_CHUNK0);
    if (next_chunk > 1) next_off += __ldg(kp.parts + p * GP_WORDS + GP_CHUNK1);
    if (next_chunk > 2) next_off += __ldg(kp.parts + p * GP_WORDS + GP_CHUNK2);
    C0 = ring_wait(ps);
    PROF(7);
    // keep the chunk table: chunk 0's slot is recycled
    const uint32_t nch = C0[PH_N_CHUNKS];
    for (uint32_t k = tid; k < nch; k += GEM_THREADS) ps.ctab[k] = C0[C0[PH_OFF_CHUNKS] + k];
    ctab = ps.ctab;
    n_pin = 0;
  }
  const uint4 h0 = *reinterpret_cast<const uint4*>(C0);
  const uint4 h1 = *(reinterpret_cast<const uint4*>(C0) + 1);
  const uint4 h2 = *(reinterpret_cast<const uint4*>(C0) + 2);
  const uint4 h3 = *(reinterpret_cast<const uint4*>(C0) + 3);
  const uint32_t n_gread = h0.y, n_layers = h0.z, n_out = h0.w;
  const uint32_t n_ram = h1.x, off_gread = h1.z, off_layers = h1.w;
  const uint32_t off_out = h2.x, off_ram = h2.y, n_out_pad = h3.x, n_chunks = h3.z;
  auto refill = [&]() {   // issue chunks into free ring slots
    if (!ps.resident)
      while (next_chunk < n_chunks && ps.seq_issue - ps.seq_free < ps.R) {
        const uint32_t words = ctab[next_chunk];
        ring_issue(ps, gprog + next_off, words);
        next_off += words;
        next_chunk++;
      }
  };
  // ---- a2: global read of input ports (once per cycle)
  // 4 entries per thread per round: all loads are issued before the stores so
  // their L2 latencies overlap
  const uint2* gr = reinterpret_cast<const uint2*>(C0 + off_gread);
  const uint32_t n_gr = n_gread * nst;
  bool changed = act_first;
  // GEM_F_ACTIVITY: used-bit masks of the gread words (the program's tail)
  const uint32_t* gmask = (ACT && act) ? gprog + __ldg(kp.parts + p * GP_WORDS + GP_PROG_LEN) - ((n_gread + 3u) & ~3u)
                              : nullptr;
  constexpr uint32_t GU = 4;   // port loads in flight per thread (8 measured slower on C3)
  for (uint32_t k0 = 0; k0 < n_gr; k0 += GU * GEM_THREADS) {
    uint32_t v[GU], dst[GU];
#pragma unroll
    for (uint32_t u = 0; u < GU; u++) {
      const uint32_t k = k0 + u * GEM_THREADS + tid;
      dst[u] = ~0u;
      if (k < n_gr) {
        const uint32_t j = k / n_gread, st = st0 + j;
        const uint2 e = gr[k - j * n_gread];
        const uint32_t reg = GEM_GID_REGION(e.x), idx = GEM_GID_INDEX(e.x);
        const uint32_t* a;
        if (reg == GEM_R_PI) a = kp.pi + ((size_t)st * kp.in_cap + kp.in_base + c) * kp.pi_words + idx;
        else if (reg == GEM_R_Q) a = kp.q + ((size_t)cur * kp.n_streams + st) * kp.q_words + idx;
        else if (reg == GEM_R_RD) a = kp.rd + ((size_t)cur * kp.n_streams + st) * kp.n_rams + idx;
        else a = kp.cut + (size_t)st * kp.cut_words + idx;
        if (LOC) {
          if (reg == GEM_R_PI) {
            v[u] = c ? (*pv)[u] : rd_global(a);
            if (c + 1 < kp.ncycles) (*pv)[u] = rd_global(a + kp.pi_words);   // cycle c+1's word
          } else if (reg == GEM_R_Q) {
            v[u] = loc[cur * kp.loc_words + idx];
          } else if (reg == GEM_R_RD) {
            v[u] = loc[cur * kp.loc_words + kp.q_words + idx];
          } else {
            v[u] = rd_global(a);
          }
        } else {
          v[u] = rd_global(a);
        }
        dst[u] = j * SW + e.y;
      }
    }
#pragma unroll
    for (uint32_t u = 0; u < GU; u++)
      if (dst[u] != ~0u) {
        if (ACT && act) {
          const uint32_t k = k0 + u * GEM_THREADS + tid;
          changed |= ((act[k] ^ v[u]) & __ldg(gmask + k)) != 0u;
          act[k] = v[u];
        } else {
          sts(s_base + 4 * dst[u], v[u]);
        }
      }
  }
  bool skip = false;
  if (ACT && act) {
    skip = __syncthreads_or(changed ? 1 : 0) == 0;
    if (!skip)
      for (uint32_t k = tid; k < n_gr; k += GEM_THREADS) sts(s_base + 4 * gr[k].y, act[k]);
    if (tid == 0) atomicAdd(kp.act_cnt + (skip ? 1 : 0), 1ull);
  }
  PROF(8);
  if (tid < nst) S[tid * SW] = 0u;
  // first layer's records (independent of S) before the barrier
  LayerRegs R;
  const uint32_t* Lres = C0 + off_layers;
  if (n_layers) {
    const uint32_t* L;
    if (1 < n_pin) { L = Lres; Lres += ctab[1]; }
    else L = ring_wait(ps);
    load_layer(L, dir0_entry(C0, h3.w), R);
  }
  PROF(9);
  __syncthreads();   // S ready; chunk 0 and layer 0's chunk consumed
  ps.seq_free = ps.seq_wait;   // records are in registers; waited slots are free
  // (the S[0] read makes the stamp wait for the barrier release, which
  // BAR.SYNC.DEFER_BLOCKING otherwise defers to the first dependent access)
  if (prof_on && tid == 0 && lds(s_base) == 0u) PROF(1);
  refill();
  // a skipped partition (GEM_F_ACTIVITY) evaluates no layer; if it streams
  // chunks it still walks the ring in the same order (kept out of the hot loop
  // below, whose code must not change when pruning is off)
  if (ACT && skip) {
    for (uint32_t l = 0; l + 1 < n_layers; l++) {
      if (!(2 + l < n_pin)) ring_wait(ps);
      __syncthreads();
      ps.seq_free = ps.seq_wait;
      refill();
    }
    __syncthreads();   // S / ramp reads below follow the port compare
    ps.seq_free = ps.seq_wait;
    refill();
  }
  // ---- a3-a5: layers, software-pipelined: layer l+1's records are loaded
  // into registers before the barrier that ends layer l
  // (the skip test stays out of the loop: a loop bound that depends on it
  // slowed the activity build's layers by ~8%)
  if (ACT && skip) goto commit;
  for (uint32_t l = 0; l < n_layers; l++) {
    // stream j uses named barrier 1 + j (group <= GEM_MAX_GROUP < 16)
    if (nst == 1 && s_base == GEM_S0_ADDR) exec_layer<true>(R, s_base, g_smem, topb, 1);
    else
      for (uint32_t j = 0; j < nst; j++)
        exec_layer<false>(R, s_base + 4 * j * SW, g_smem + j * SW, topb + 16 * j, 1 + j);
    const bool ptop = (R.flags & GEM_LF_USES_TOP) != 0;
    const uint32_t ptopc = R.topc, ptopwo = R.topwo;
    if (l + 1 < n_layers) {
      const uint32_t* L;
      if (2 + l < n_pin) { L = Lres; Lres += ctab[2 + l]; }
      else L = ring_wait(ps);
      load_layer(L, R.ndir, R);
    }
    if (ptop && warp == 0)
      for (uint32_t j = 0; j < nst; j++) top_layer(ptopc, ptopwo, s_base + 4 * j * SW, topb + 16 * j, 1 + j);
    __syncthreads();
    ps.seq_free = ps.seq_wait;
    refill();
  }
commit:
  PROF(2);
  // ---- a6: endpoint commit (warp ballot-gather per output word and stream)
  const uint32_t* od = n_layers + 1 < n_pin ? (C0 + off_out) : ring_wait(ps);
  const uint32_t* os = od + n_out_pad;
  for (uint32_t jj = warp; jj < n_out * nst; jj += GEM_WARPS) {
    const uint32_t j = jj / n_out, o = jj - j * n_out, st = st0 + j;
    const uint32_t e = os[o * 32 + lane];
    const uint32_t src = e & 0x7FFFFFFFu;
    const uint32_t bit = ((S[j * SW + (src >> 5)] >> (src & 31u)) & 1u) ^ (e >> 31);
    const uint32_t v = __ballot_sync(0xFFFFFFFFu, bit);
    if (lane == 0) {
      const uint32_t dst = od[o];
      const uint32_t reg = GEM_GID_REGION(dst), idx = GEM_GID_INDEX(dst);
      if (reg == GEM_R_Q) {
        const size_t o = ((size_t)nxt * kp.n_streams + st) * kp.q_words + idx;
        __stcg(kp.q + o, v);
        if (LOC) loc[nxt * kp.loc_words + idx] = v;
        if (DIST) dist_put(kp, kp.peer_q, o, v);
      } else if (reg == GEM_R_PO) {
        const size_t o = ((size_t)st * kp.out_cap + c) * kp.po_words + idx;
        __stcg(kp.po + o, v);
        if (DIST) dist_put(kp, kp.peer_po, o, v);
      } else if (reg == GEM_R_CUT) {
        const size_t o = (size_t)st * kp.cut_words + idx;
        __stcg(kp.cut + o, v);
        if (DIST) dist_put(kp, kp.peer_cut, o, v);
      } else {
        ramp[j * 4 * GEM_MAX_RAMS_PER_PART + idx] = v;
      }
    }
  }
  PROF(11);
  // ---- a7: RAM blocks (read-first, then per-bit write; readings U7-U10)
  if (n_ram) {
    __syncthreads();
    const uint32_t* rr = od + (off_ram - off_out);
    for (uint32_t jr = tid; jr < n_ram * nst; jr += GEM_THREADS) {
      const uint32_t j = jr / n_ram, r = jr - j * n_ram, st = st0 + j;
      const uint32_t* rp = ramp + j * 4 * GEM_MAX_RAMS_PER_PART + 4 * r;
      const uint32_t id = rr[4 * r];
      const uint32_t ra = rp[GEM_PORT_RADDR] & (GEM_RAM_WORDS - 1);
      const uint32_t wa = rp[GEM_PORT_WADDR] & (GEM_RAM_WORDS - 1);
      const uint32_t wd = rp[GEM_PORT_WDATA], be = rp[GEM_PORT_WBE];
      uint32_t* M = kp.mem + ((size_t)st * kp.n_rams + id) * GEM_RAM_WORDS;
      const uint32_t old = __ldcg(M + ra);
      const uint32_t cur_w = __ldcg(M + wa);
      __stcg(M + wa, (cur_w & ~be) | (wd & be));
      const size_t o = ((size_t)nxt * kp.n_streams + st) * kp.n_rams + id;
      __stcg(kp.rd + o, old);
      if (LOC) loc[nxt * kp.loc_words + kp.q_words + id] = old;
      if (DIST) dist_put(kp, kp.peer_rd, o, old);
    }
  }
  __syncthreads();  // S / ramp / ring slots reused by the next work item
  ps.seq_free = ps.seq_issue;   // every chunk of this item consumed
  PROF(3);
  if (prof_on && tid == 0) {
    kp.prof[((size_t)c * gridDim.x + blockIdx.x) * GEM_PROF_SLOTS + 6] = n_layers;
    kp.prof[((size_t)c * gridDim.x + blockIdx.x) * GEM_PROF_SLOTS + 10] = p;
  }
}

// Parity instruments: trace / digest of Q(t+1) in external (AIGER) order.
__device__ void record_state(const KParams& kp, uint32_t c, uint32_t buf) {
  const uint32_t total = kp.n_streams * kp.q_ext_words;
  for (uint32_t g = blockIdx.x * blockDim.x + threadIdx.x; g < total; g += gridDim.x * blockDim.x) {
    const uint32_t st = g / kp.q_ext_words, w = g % kp.q_ext_words;
    const uint32_t* Q = kp.q + ((size_t)buf * kp.n_streams + st) * kp.q_words;
    uint32_t v = 0;
    for (uint32_t b = 0; b < 32; b++) {
      const uint32_t e = w * 32 + b;
      if (e >= kp.n_flops) break;
      const uint32_t i = __ldg(kp.q_int_of_ext + e);
      v |= ((__ldcg(Q + (i >> 5)) >> (i & 31u)) & 1u) << b;
    }
    if (kp.flags & GEM_F_TRACE_STATE) kp.q_trace[((size_t)st * kp.out_cap + c) * kp.q_ext_words + w] = v;
    if (kp.flags & GEM_F_DIGEST) {
      const uint32_t r = w & 63u;
      const unsigned long long x = (unsigned long long)v;
      const unsigned long long rot = r ? ((x << r) | (x >> (64 - r))) : x;
      atomicAdd(kp.digest + (size_t)st * kp.out_cap + c, rot * (2ull * w + 1ull));
    }
  }
}

// ACT: GEM_F_ACTIVITY build of the kernel (the plain one carries no pruning code);
// LOC: single-CTA launch, flops / RAM-read words in shared memory; DIST: one
// rank of a design split over devices (peer stores + cross-device barrier)
template <bool ACT, bool LOC, bool DIST>
__global__ void __launch_bounds__(GEM_THREADS, 2) gem_step_kernel(const KParams kp) {
  extern __shared__ __align__(16) uint32_t smem[];
  // layout (words): S[group][state_words] | area[area_words] | ctab[256] | ramp[group][128] |
  //                 topb[group][16] | res_p[16] | res_off[16] | res_n[16] | wl cache | mbar[16 x u64] |
  //                 act[act_words]
  // S must stay at offset 0 (leaf entries carry byte offsets into it).
  uint32_t* S = smem;
  uint32_t* area = S + kp.group * kp.state_words;
  uint32_t* ctab = area + kp.area_words;
  uint32_t* ramp = ctab + GEM_MAX_CHUNKS;
  uint32_t* topb = ramp + kp.group * 4 * GEM_MAX_RAMS_PER_PART;
  uint32_t* res_p = topb + 16 * kp.group;
  uint32_t* res_off = res_p + GEM_MAX_RESIDENT;
  uint32_t* res_n = res_off + GEM_MAX_RESIDENT;      // [0] n_res, [1] resident, [2..4] pinned chunks/words, ring R
  // work-list cache: [0,8) stage begins, [8,16) stage ends, [16,24) cache base
  // per stage, [24] cached flag, [32, 32 + 2*GEM_WL_CACHE) items (uint2)
  uint32_t* wlc = res_n + 16;
  uint64_t* mbar = reinterpret_cast<uint64_t*>(wlc + GEM_WL_CACHE_WORDS);
  uint32_t* act_buf = reinterpret_cast<uint32_t*>(mbar + 16);  // [act_words] (GEM_F_ACTIVITY)
  uint32_t* loc = act_buf + kp.act_words;                        // [2][loc_words] (LOC kernels)
  const uint32_t tid = threadIdx.x;
  const uint32_t G = gridDim.x, B = blockIdx.x;
  if (tid == 0) {
    // the CTA's work list is fixed for the launch: keep it in shared memory
    // (saves two dependent global loads at the start of every cycle)
    uint32_t n = 0;
    bool ok = kp.n_stages <= GEM_WL_MAX_STAGES;
    for (uint32_t s = 0; s < kp.n_stages && ok; s++) {
      const uint32_t b = __ldg(kp.wl_off + s * (G + 1) + B), e = __ldg(kp.wl_off + s * (G + 1) + B + 1);
      wlc[s] = b;
      wlc[8 + s] = e;
      wlc[16 + s] = n;
      if (n + (e - b) > GEM_WL_CACHE) { ok = false; break; }
      for (uint32_t k = b; k < e; k++) reinterpret_cast<uint2*>(wlc + 32)[n++] = __ldg(&kp.wl_items[k]);
    }
    wlc[24] = ok ? 1u : 0u;
  }
  __syncthreads();
  const bool wl_cached = wlc[24] != 0;
  auto wl_begin = [&](uint32_t s) { return wl_cached ? wlc[s] : __ldg(kp.wl_off + s * (G + 1) + B); };
  auto wl_end = [&](uint32_t s) { return wl_cached ? wlc[8 + s] : __ldg(kp.wl_off + s * (G + 1) + B + 1); };
  auto wl_item = [&](uint32_t s, uint32_t k) -> uint2 {
    return wl_cached ? reinterpret_cast<const uint2*>(wlc + 32)[wlc[16 + s] + (k - wlc[s])] : __ldg(&kp.wl_items[k]);
  };
  for (uint32_t k = tid; k < 16 * kp.group; k += GEM_THREADS) topb[k] = 0u;
  if (tid == 0) {
    for (uint32_t k = 0; k <= GEM_RING_MAX; k++) mbar_init(mbar + k, 1);
    fence_mbar_init();
    // residency: the distinct partitions of this CTA's work lists (fixed for the launch)
    uint32_t n = 0, words = 0;
    bool ok = kp.allow_resident != 0;
    for (uint32_t s = 0; s < kp.n_stages && ok; s++) {
      for (uint32_t k = wl_begin(s); k < wl_end(s); k++) {
        const uint32_t p = wl_item(s, k).x;
        bool seen = false;
        for (uint32_t j = 0; j < n; j++) seen |= res_p[j] == p;
        if (seen) continue;
        const uint32_t len = (__ldg(kp.parts + p * GP_WORDS + GP_PROG_LEN) + 3u) & ~3u;
        if (n == GEM_MAX_RESIDENT || words + len > kp.area_words) { ok = false; break; }
        res_p[n] = p;
        res_off[n] = words;
        words += len;
        n++;
      }
    }
    res_n[0] = n;
    res_n[1] = ok ? 1u : 0u;
    res_n[2] = 0u;               // pinned chunks
    res_n[3] = 0u;               // pinned words
    res_n[4] = kp.ring_slots;    // ring depth
    if (!ok && kp.allow_resident) {
      // pinned prefix: a CTA that runs a single partition whose program does
      // not fit keeps its leading chunks (header, gread list, first layers)
      // for the whole launch and streams only the rest through a ring
      uint32_t p1 = ~0u;
      bool single = true;
      for (uint32_t s = 0; s < kp.n_stages; s++)
        for (uint32_t k = wl_begin(s); k < wl_end(s); k++) {
          const uint32_t p = wl_item(s, k).x;
          if (p1 == ~0u) p1 = p;
          else single &= p == p1;
        }
      if (single && p1 != ~0u) {
        const uint32_t* g = kp.prog + __ldg(kp.parts + p1 * GP_WORDS + GP_PROG_OFF);
        const uint32_t nch = min(__ldg(g + PH_N_CHUNKS), (uint32_t)GEM_MAX_CHUNKS), offc = __ldg(g + PH_OFF_CHUNKS);
        // ring slots sized for the largest chunk that still streams (the
        // light tail layers are a fraction of the heaviest), so the ring is
        // as deep as possible: ctab (unused in this mode) holds suffix maxima
        for (uint32_t k = nch; k-- > 0;) ctab[k] = max(__ldg(g + offc + k), k + 1 < nch ? ctab[k + 1] : 0u);
        uint32_t P = 0, pw = 0;
        while (P < nch) {
          const uint32_t sz = __ldg(g + offc + P);
          const uint32_t rest = P + 1 < nch ? ctab[P + 1] : 0u;
          if (pw + sz + 2 * rest > kp.area_words) break;
          pw += sz;
          P++;
        }
        if (P >= 2) {
          const uint32_t slot = P < nch ? ((ctab[P] + 3u) & ~3u) : 4u;
          uint32_t R = 2;
          while (2 * R <= GEM_RING_MAX && pw + 2 * R * slot <= kp.area_words) R *= 2;
          res_n[2] = P;
          res_n[3] = pw;
          res_n[4] = R;
          res_n[5] = slot;
          mbar_expect_tx(mbar + GEM_RING_MAX, pw * 4);
          tma_load_1d(area, g, pw * 4, mbar + GEM_RING_MAX);
        }
      }
    }
    if (ok && words) {
      mbar_expect_tx(mbar + GEM_RING_MAX, words * 4);
      for (uint32_t k = 0; k < n; k++) {
        const uint32_t p = res_p[k];
        const uint32_t len = (__ldg(kp.parts + p * GP_WORDS + GP_PROG_LEN) + 3u) & ~3u;
        tma_load_1d(area + res_off[k], kp.prog + __ldg(kp.parts + p * GP_WORDS + GP_PROG_OFF), len * 4,
                    mbar + GEM_RING_MAX);
      }
    }
  }
  __syncthreads();
  ProgSrc ps;
  ps.mbar = mbar;
  ps.area = area;
  ps.ctab = ctab;
  ps.resident = res_n[1] != 0;
  ps.n_res = res_n[0];
  ps.res_p = res_p;
  ps.res_off = res_off;
  ps.slot_words = kp.slot_words;
  ps.R = kp.ring_slots;
  ps.seq_issue = 0;
  ps.seq_wait = 0;
  ps.seq_free = 0;
  ps.pin_chunks = res_n[2];
  ps.pin_off = res_n[3];
  ps.l2pol = kp.l2_frac > 0.f ? l2_policy(kp.l2_frac) : l2_policy_unchanged();
  ps.pin = area;
  ps.pro_chunk = ps.pro_off = 0;
  if (ps.pin_chunks) {
    ps.area = area + ps.pin_off;   // ring after the pinned prefix
    ps.R = res_n[4];
    ps.slot_words = res_n[5];
  }
  if ((ps.resident && ps.n_res) || ps.pin_chunks) mbar_wait(mbar + GEM_RING_MAX, 0);
  // first work item of this CTA in a cycle: partition id, or ~0u
  auto first_part = [&]() -> uint32_t {
    for (uint32_t s = 0; s < kp.n_stages; s++)
      if (wl_begin(s) < wl_end(s)) return wl_item(s, wl_begin(s)).x;
    return ~0u;
  };
  auto prologue = [&](uint32_t p) {
    if (ps.pin_chunks) issue_prologue_pinned(kp, ps, p);
    else issue_prologue(kp, ps, p);
  };
  if (!ps.resident && kp.ncycles) {
    const uint32_t p0 = first_part();
    if (p0 != ~0u) prologue(p0);
  }
  // activity pruning: only a CTA with exactly one work item (one partition,
  // one stream) per cycle keeps S, ramp and the port copy from cycle to cycle
  uint32_t* act = nullptr;
  if (ACT && kp.act_words && kp.group == 1) {
    uint32_t n_it = 0;
    for (uint32_t s = 0; s < kp.n_stages; s++) n_it += wl_end(s) - wl_begin(s);
    if (n_it == 1) act = act_buf;
  }

  unsigned long long bar_target = 0;
  const bool instr = (kp.flags & (GEM_F_TRACE_STATE | GEM_F_DIGEST)) != 0;
  uint32_t pv[4] = {0u, 0u, 0u, 0u};   // LOC: prefetched PI words of the next cycle
  if (LOC) {
    // the state of cycle t0 into shared memory (Q[cur] and RD[cur] of the launch's first cycle)
    const uint32_t c0 = (uint32_t)(kp.t0 & 1u);
    for (uint32_t k = tid; k < kp.loc_words; k += GEM_THREADS)
      loc[c0 * kp.loc_words + k] = k < kp.q_words ? __ldcg(kp.q + (size_t)c0 * kp.n_streams * kp.q_words + k)
                                                  : __ldcg(kp.rd + (size_t)c0 * kp.n_streams * kp.n_rams + (k - kp.q_words));
    __syncthreads();
  }
  // DIST: no rank stores into a peer's buffers before every rank has started
  // this launch (a peer may still be reading the previous launch's outputs)
  if (DIST) grid_sync<true>(kp, bar_target);
  for (uint32_t c = 0; c < kp.ncycles; c++) {
    const uint64_t t = kp.t0 + c;
    const uint32_t cur = (uint32_t)(t & 1u), nxt = cur ^ 1u;
    if (instr && c > 0) record_state(kp, c - 1, cur);
    const bool prof_on = kp.prof && c < kp.prof_cycles;
    PROF(0);
    for (uint32_t s = 0; s < kp.n_stages; s++) {
      const uint32_t kb = wl_begin(s), ke = wl_end(s);
      for (uint32_t k = kb; k < ke; k++) {
        const uint2 it = wl_item(s, k);
        const uint32_t nst = min(kp.group, kp.n_streams - it.y);
        run_partition<ACT, LOC, DIST>(kp, ps, S, ramp, topb, it.x, it.y, nst, c, cur, nxt, prof_on && k == kb && s == 0,
                                act, c == 0, loc, &pv);
        if (!ps.resident) {
          // prefetch the next work item's prologue (overlaps the grid barrier)
          uint32_t np = ~0u;
          if (k + 1 < ke) np = wl_item(s, k + 1).x;
          for (uint32_t s2 = s + 1; np == ~0u && s2 < kp.n_stages; s2++)
            if (wl_begin(s2) < wl_end(s2)) np = wl_item(s2, wl_begin(s2)).x;
          if (np == ~0u && c + 1 < kp.ncycles) np = first_part();
          if (np != ~0u) prologue(np);
        }
      }
      if (s == 0) PROF(4);
      grid_sync<DIST>(kp, bar_target);
    }
    PROF(5);
  }
  if (instr) record_state(kp, kp.ncycles - 1, (uint32_t)((kp.t0 + kp.ncycles) & 1u));
}

// ---- lane-mode prologue helpers (same protocol as issue_prologue, lane fields)
#include "gem_lanes.cuh"
#include "gem_words.cuh"


// ---- latency-floor microbenchmarks (bench.py roofline; not on the hot path)
// Minimal layer: the dependent chain every layer must traverse even with one
// leaf per thread: one gathered LDS, levels 1-5 in-thread, warp ballot, levels
// 6-10, named-barrier hand-off of levels 11-13 to warp 0, write-out, barrier.
__global__ void __launch_bounds__(GEM_THREADS, 1) floor_layer_kernel(unsigned long long* out, uint32_t iters) {
  __shared__ uint32_t S[2048];
  __shared__ uint32_t topb[8];
  const uint32_t tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  for (uint32_t i = tid; i < 2048; i += GEM_THREADS) S[i] = i * 2654435761u;
  __syncthreads();
  const uint32_t base = smem_u32(S);
  uint32_t x = tid;
  const unsigned long long t0 = clock64();
  for (uint32_t it = 0; it < iters; it++) {
    const uint32_t v = lds(base + 4 * ((x ^ it) & 2047u));
    const uint32_t P = fold5(v, 0x1234567u, 0x89ABCDEu, 0x5555u);
    const uint32_t u = __ballot_sync(0xFFFFFFFFu, (P >> 30) & 1u);
    const uint32_t Pw = fold5(u, 0x7654321u, 0x0FEDCBAu, 0x3333u);
    if (lane == 0) topb[warp] = (Pw >> 30) & 1u;
    if (warp != 0) {
      asm volatile("bar.arrive 1, %0;" ::"r"(GEM_THREADS) : "memory");
    } else {
      asm volatile("bar.sync 1, %0;" ::"r"(GEM_THREADS) : "memory");
      if (lane == 0) {
        uint32_t t8 = 0;
        for (uint32_t w = 0; w < GEM_WARPS; w++) t8 |= topb[w] << w;
        sts(base + 4 * (1024 + (it & 1023)), fold3(t8, 0x55u, 0x33u, 0x0Fu));
      }
    }
    __syncthreads();
    x = P ^ Pw ^ lds(base + 4 * (1024 + (it & 1023)));
  }
  const unsigned long long t1 = clock64();
  if (tid == 0) out[0] = (t1 - t0) / iters;
  if (x == 0x9E3779B9u) out[1] = x;   // keep the chain live
}

// Minimal word-mode step (gem_words.cuh): after the block barrier every thread
// loads two operand words (bank-conflict-free), computes the AND with its
// inversions and stores the result, then the next barrier -- the dependent
// chain every step traverses however few ops it has.  Op words stay in
// registers (the kernel prefetches them off the chain).
__global__ void __launch_bounds__(GEM_THREADS, 1) floor_step_kernel(unsigned long long* out, uint32_t iters) {
  __shared__ uint32_t S[2048];
  const uint32_t tid = threadIdx.x;
  for (uint32_t i = tid; i < 2048; i += GEM_THREADS) S[i] = i * 2654435761u;
  __syncthreads();
  const uint32_t base = smem_u32(S);
  uint32_t a_off = 4 * (tid & 1023u), b_off = 4 * (1024 + ((tid + 7) & 1023u));
  const unsigned long long t0 = clock64();
  for (uint32_t it = 0; it < iters; it++) {
    const uint32_t a = lds(base + a_off), b = lds(base + b_off);
    const uint32_t r = (a ^ it) & (b ^ (it >> 1));
    sts(base + 4 * (((tid + 32 * (it & 7)) & 1023u) + 1024 * (it & 1)), r);
    __syncthreads();
    a_off ^= 4096u;   // next step reads the words this one wrote
    b_off ^= 4096u;
  }
  const unsigned long long t1 = clock64();
  if (tid == 0) out[0] = (t1 - t0) / iters;
}

// Grid barrier round trip at a given grid size (same grid_sync as the kernels).
__global__ void __launch_bounds__(GEM_THREADS, 1) floor_barrier_kernel(const KParams kp, unsigned long long* out,
                                                                       uint32_t iters) {
  unsigned long long epoch = 0;
  grid_sync(kp, epoch);
  const unsigned long long t0 = clock64();
  for (uint32_t it = 0; it < iters; it++) grid_sync(kp, epoch);
  const unsigned long long t1 = clock64();
  if (blockIdx.x == 0 && threadIdx.x == 0) out[0] = (t1 - t0) / iters;
}

// external <-> internal layout conversion kernels
// out[st][row][ext_w] = gather of 32 internal bits via int_of_ext
__global__ void unpermute_kernel(const uint32_t* __restrict__ in, uint32_t* __restrict__ out,
                                 const uint32_t* __restrict__ int_of_ext, uint32_t n_bits, uint32_t in_words,
                                 uint32_t out_words, uint64_t rows, uint64_t in_row_stride,
                                 uint64_t out_row_stride, uint64_t rows_per_group = ~0ull,
                                 uint64_t in_group_stride = 0) {
  // input row r lives at (r / rows_per_group) * in_group_stride + (r % rows_per_group) * in_row_stride
  // (all streams of a read in one launch: groups = streams, rows = cycles)
  const uint64_t total = rows * out_words;
  for (uint64_t g = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; g < total;
       g += (uint64_t)gridDim.x * blockDim.x) {
    const uint64_t row = g / out_words;
    const uint32_t w = (uint32_t)(g % out_words);
    const uint64_t grp = row / rows_per_group, rr = row - grp * rows_per_group;
    const uint32_t* src = in + grp * in_group_stride + rr * in_row_stride;
    uint32_t v = 0;
    for (uint32_t b = 0; b < 32; b++) {
      const uint32_t e = w * 32 + b;
      if (e >= n_bits) break;
      const uint32_t i = int_of_ext[e];
      v |= ((src[i >> 5] >> (i & 31u)) & 1u) << b;
    }
    out[row * out_row_stride + w] = v;
    (void)in_words;
  }
}

// internal word = gather from external bits via ext_of_int (0xFFFFFFFF = padding -> 0)
__global__ void permute_kernel(const uint32_t* __restrict__ ext, uint32_t* __restrict__ in,
                               const uint32_t* __restrict__ ext_of_int, uint32_t int_words, uint32_t ext_words,
                               uint32_t rows) {
  const uint64_t total = (uint64_t)rows * int_words;
  for (uint64_t g = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; g < total;
       g += (uint64_t)gridDim.x * blockDim.x) {
    const uint64_t row = g / int_words;
    const uint32_t w = (uint32_t)(g % int_words);
    uint32_t v = 0;
    for (uint32_t b = 0; b < 32; b++) {
      const uint32_t e = ext_of_int[w * 32 + b];
      if (e == 0xFFFFFFFFu) continue;
      v |= ((ext[row * ext_words + (e >> 5)] >> (e & 31u)) & 1u) << b;
    }
    in[row * int_words + w] = v;
  }
}

}  // namespace

// ============================================================== host side
struct gem_sim {
  int device = 0;
  cudaStream_t stream = nullptr;
  bool own_stream = false;
  bool poisoned = false;
  uint32_t flags = 0, n_streams = 1, grid = 0, blocks_per_sm = 0, smem_bytes = 0, sm_count = 0;
  // header
  uint32_t n_pi = 0, n_po = 0, n_flops = 0, n_rams = 0, n_parts = 0, n_stages = 0, max_layers = 0,
           total_layers = 0, state_words = 0, pi_words = 0, po_words_int = 0, q_words_int = 0, cut_words = 0;
  uint32_t po_words_ext = 0, q_words_ext = 0;
  uint64_t n_and = 0, n_and_mapped = 0, program_bytes = 0;
  uint32_t max_items = 0;
  uint32_t area_words = 0, slot_words = 0, ring_slots = 0, resident = 0, group = 1;
  // lane mode (stream-sliced, >= 32 streams and a blob with lane programs)
  uint32_t act_words = 0;                      // GEM_F_ACTIVITY: max n_gread over partitions
  bool local = false;                          // single-CTA launch: LOC kernel (flops in shared memory)
  uint32_t loc_words = 0, max_gread = 0;
  uint4* d_dyn_units = nullptr;                // lane mode dynamic work units
  uint32_t n_units = 0, *d_dyn_ctr = nullptr;
  unsigned long long* d_act = nullptr;         // {evaluated, skipped}
  // word mode (single-stream latency path, WRD1 programs resident in shared memory)
  bool words = false;
  uint32_t word_state = 0, *d_wprog = nullptr;
  std::vector<uint32_t> h_wprog_len;           // [n_parts] word program lengths (words)
  uint32_t lanes = 0, n_groups = 0, lane_words = 0, lane_max_chunk = 0, ramp_words = 0, lane_groups = 1;
  bool lane_v2 = false;                        // compacted lane programs ("LAN2")
  uint32_t lane_m = 1;                         // LAN2: ops per thread and step
  uint32_t *d_lprog = nullptr, *d_pi_lane = nullptr, *d_po_lane = nullptr;
  std::vector<uint32_t> h_parts, h_stage;
  // device buffers
  uint32_t *d_prog = nullptr, *d_parts = nullptr, *d_stage = nullptr;
  uint32_t *d_q_int_of_ext = nullptr, *d_q_ext_of_int = nullptr, *d_po_int_of_ext = nullptr;
  uint32_t *d_q = nullptr, *d_rd = nullptr, *d_cut = nullptr, *d_mem = nullptr;
  uint32_t *d_pi = nullptr, *d_po = nullptr, *d_qtrace = nullptr, *d_scratch = nullptr, *d_wl_off = nullptr;
  uint2* d_wl_items = nullptr;
  unsigned long long *d_digest = nullptr, *d_bar = nullptr, *d_prof = nullptr;
  uint32_t prof_cycles = 0;
  uint32_t* h_err = nullptr;   // watchdog word (GEM_ERR_BARRIER once fired): mapped pinned host memory
  uint32_t* d_err = nullptr;   // device alias of h_err
  gem_config cfg{};            // launch tuning (include/gem.h)
  uint32_t in_cap = 0, in_queued = 0, in_head = 0, out_cap = 0, last_cycles = 0;
  size_t scratch_bytes = 0;
  uint64_t cycle = 0;
  cudaEvent_t ev0 = nullptr, ev1 = nullptr, ev_in = nullptr;
  float last_ms = 0.f;
  // single-design multi-GPU (gem_dist_*)
  uint32_t dist_world = 1, dist_rank = 0;
  std::vector<uint32_t> owner;                 // [n_parts] rank of each partition (dist only)
  bool dist_exported = false, dist_connected = false;
  unsigned long long* d_dist_flags = nullptr;  // [GEM_DIST_MAX] slots of GEM_BAR_STRIDE u64
  unsigned long long dist_epoch = 0;           // cross-device barriers completed by earlier launches
  gem_dist_buffers peers[GEM_DIST_MAX]{};
  std::vector<void*> ipc_opened;               // peer buffers mapped by gem_dist_ipc_open
};

static int fail(int code, const std::string& msg) {
  g_err = msg;
  return code;
}

// The grid-barrier watchdog's report (mapped pinned words written before the
// trap), appended to the CUDA error of the failed call.
static std::string watchdog_msg(const gem_sim* sim) {
  if (!sim || !sim->h_err || *(const volatile uint32_t*)sim->h_err != GEM_ERR_BARRIER) return "";
  return "; grid-barrier watchdog: a CTA waited > 10 s at a grid barrier (persistent grid not co-resident?)";
}

#define CK(call)                                                                          \
  do {                                                                                    \
    cudaError_t e_ = (call);                                                              \
    if (e_ != cudaSuccess) {                                                              \
      if (sim) sim->poisoned = true;                                                      \
      return fail(e_ == cudaErrorMemoryAllocation ? GEM_E_NOMEM : GEM_E_CUDA,             \
                  std::string(#call) + ": " + cudaGetErrorString(e_) + watchdog_msg(sim)); \
    }                                                                                     \
  } while (0)

template <class T>
static cudaError_t dalloc(T** p, size_t bytes) {
  return cudaMalloc((void**)p, std::max<size_t>(bytes, 16));
}

static int ensure_scratch(gem_sim* sim, size_t bytes) {
  if (sim->scratch_bytes >= bytes) return 0;
  if (sim->d_scratch) cudaFree(sim->d_scratch);
  sim->d_scratch = nullptr;
  sim->scratch_bytes = 0;
  CK(dalloc(&sim->d_scratch, bytes));
  sim->scratch_bytes = bytes;
  return 0;
}

static int ensure_out(gem_sim* sim, uint32_t ncycles) {
  if (sim->out_cap >= ncycles && sim->d_po) return 0;
  if (sim->dist_exported)   // peers hold pointers into d_po
    return fail(GEM_E_INVAL, "more cycles per gem_step than gem_dist_export's max_cycles");
  uint32_t cap = std::max<uint32_t>(ncycles, 16);
  if (sim->d_po) cudaFree(sim->d_po);
  if (sim->d_qtrace) cudaFree(sim->d_qtrace);
  if (sim->d_digest) cudaFree(sim->d_digest);
  sim->d_po = nullptr; sim->d_qtrace = nullptr; sim->d_digest = nullptr;
  sim->out_cap = 0;
  CK(dalloc(&sim->d_po, (size_t)sim->n_streams * cap * sim->po_words_int * 4));
  if (sim->lanes) {
    if (sim->d_po_lane) cudaFree(sim->d_po_lane);
    sim->d_po_lane = nullptr;
    CK(dalloc(&sim->d_po_lane, (size_t)cap * sim->po_words_int * 32 * sim->n_groups * 4));
  }
  if (sim->flags & GEM_F_TRACE_STATE) CK(dalloc(&sim->d_qtrace, (size_t)sim->n_streams * cap * sim->q_words_ext * 4));
  if (sim->flags & GEM_F_DIGEST) CK(dalloc(&sim->d_digest, (size_t)sim->n_streams * cap * 8));
  sim->out_cap = cap;
  return 0;
}

static int check(const gem_sim* sim) {
  if (!sim) return fail(GEM_E_INVAL, "null handle");
  if (sim->poisoned) return fail(GEM_E_CUDA, "handle poisoned by an earlier CUDA error");
  return 0;
}

// Longest-processing-time-first work lists: per stage, the (partition, stream)
// items sorted by the mapper's cost estimate are assigned one by one to the
// least-loaded CTA.  Returns the estimated makespan (sum over stages).
static double build_worklists(const gem_sim* sim, uint32_t G, std::vector<uint32_t>& off,
                              std::vector<uint2>& items) {
  off.assign((size_t)sim->n_stages * (G + 1), 0);
  items.clear();
  double makespan = 0;
  for (uint32_t s = 0; s < sim->n_stages; s++) {
    const uint32_t pb = sim->h_stage[s], np = sim->h_stage[s + 1] - pb;
    // a scheduling unit = `run` consecutive stream groups of one partition, kept
    // together on one CTA (lane mode: consecutive items then share the
    // partition's input-port list and program in L1/L2)
    // (word mode: every stream of a partition on one CTA, so its program is
    // resident once)
    const uint32_t run = sim->lanes ? (sim->cfg.lane_run ? sim->cfg.lane_run : 4u) : sim->words ? sim->n_streams : 1u;
    std::vector<std::pair<uint32_t, uint2>> its;
    its.reserve((size_t)np * sim->n_streams);
    for (uint32_t st = 0; st < sim->n_streams; st += sim->group * run)
      for (uint32_t k = 0; k < np; k++) {
        const uint32_t p = sim->h_stage[sim->n_stages + 1 + pb + k];
        if (!sim->owner.empty() && sim->owner[p] != sim->dist_rank) continue;   // another rank's
        const uint32_t nst = std::min(sim->group * run, sim->n_streams - st);
        const uint32_t n_items = (nst + sim->group - 1) / sim->group;
        const double c = sim->h_parts[(size_t)p * GP_WORDS + GP_COST] *
                         (run > 1 ? (double)n_items : (1.0 + 0.7 * (nst - 1)));
        its.push_back({(uint32_t)std::min(c, 4.0e9), make_uint2(p, st)});
      }
    std::stable_sort(its.begin(), its.end(), [](const std::pair<uint32_t, uint2>& x,
                                                const std::pair<uint32_t, uint2>& y) { return x.first > y.first; });
    std::vector<std::vector<uint2>> lists(G);
    // min-heap of (load, cta)
    std::vector<std::pair<double, uint32_t>> heap;
    for (uint32_t b = 0; b < G; b++) heap.push_back({0.0, b});
    auto cmp = [](const std::pair<double, uint32_t>& x, const std::pair<double, uint32_t>& y) {
      return x.first > y.first || (x.first == y.first && x.second > y.second);
    };
    std::make_heap(heap.begin(), heap.end(), cmp);
    double mx = 0;
    for (auto& it : its) {
      std::pop_heap(heap.begin(), heap.end(), cmp);
      auto& h = heap.back();
      for (uint32_t r = 0; r < run; r++) {
        const uint32_t st = it.second.y + r * sim->group;
        if (st >= sim->n_streams) break;
        lists[h.second].push_back(make_uint2(it.second.x, st));
      }
      h.first += std::max<uint32_t>(it.first, 1);
      mx = std::max(mx, h.first);
      std::push_heap(heap.begin(), heap.end(), cmp);
    }
    makespan += mx;
    uint32_t* o = &off[(size_t)s * (G + 1)];
    for (uint32_t b = 0; b < G; b++) {
      o[b] = (uint32_t)items.size();
      items.insert(items.end(), lists[b].begin(), lists[b].end());
    }
    o[G] = (uint32_t)items.size();
  }
  return makespan;
}

static const void* step_kernel_for(const gem_sim* sim) {
  if (sim->dist_world > 1) return (const void*)gem_step_kernel<false, false, true>;
  if (sim->act_words) return (const void*)gem_step_kernel<true, false, false>;
  return sim->local ? (const void*)gem_step_kernel<false, true, false> : (const void*)gem_step_kernel<false, false, false>;
}

// Choose CTAs per SM, grid, work lists and the shared-memory program mode.
// Resident mode (every program a CTA runs copied into its shared memory once
// per launch) is used when it fits; otherwise programs stream through a TMA
// ring of >= 2 slots.  Single-stream (latency) runs prefer one CTA per SM so
// the critical partitions do not share an SM; GEM_BPS=n overrides.
static int plan_launch(gem_sim* sim, uint32_t max_chunk_words, uint32_t grid_limit) {
  int sms = 0, coop = 0, optin = 0, per_sm = 0;
  CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, sim->device));
  CK(cudaDeviceGetAttribute(&coop, cudaDevAttrCooperativeLaunch, sim->device));
  CK(cudaDeviceGetAttribute(&optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, sim->device));
  CK(cudaDeviceGetAttribute(&per_sm, cudaDevAttrMaxSharedMemoryPerMultiprocessor, sim->device));
  if (!coop) return fail(GEM_E_UNSUPPORTED, "device lacks cooperative launch");
  sim->sm_count = (uint32_t)sms;
  const uint32_t slot = (max_chunk_words + 3u) & ~3u;
  // streams per work item: as many stream states as fit beside a 3-slot ring
  sim->group = 1;
  if (sim->n_streams > 1) {
    uint32_t g = sim->cfg.max_group ? sim->cfg.max_group : GEM_MAX_GROUP;
    g = std::max<uint32_t>(1, std::min<uint32_t>(std::min<uint32_t>(g, GEM_MAX_GROUP), sim->n_streams));
    while (g > 1 && (uint64_t)(g * (sim->state_words + 4 * GEM_MAX_RAMS_PER_PART + 16) + GEM_MAX_CHUNKS + 96 + GEM_WL_CACHE_WORDS +
                               3 * slot) * 4 > (uint64_t)optin)
      g /= 2;
    sim->group = g;
  }
  sim->max_items = 0;
  for (uint32_t s = 0; s < sim->n_stages; s++) {
    uint32_t np = sim->h_stage[s + 1] - sim->h_stage[s];
    if (!sim->owner.empty()) {   // dist: this rank's partitions only
      np = 0;
      for (uint32_t k = sim->h_stage[s]; k < sim->h_stage[s + 1]; k++)
        np += sim->owner[sim->h_stage[sim->n_stages + 1 + k]] == sim->dist_rank;
    }
    sim->max_items = std::max(sim->max_items, np * ((sim->n_streams + sim->group - 1) / sim->group));
  }
  if (sim->group != 1) sim->act_words = 0;   // activity pruning needs one stream per work item
  // one partition, one stream, one stage: a single CTA owns every flop and RAM,
  // so the LOC kernel keeps them in shared memory across cycles
  sim->loc_words = sim->q_words_int + sim->n_rams;
  sim->local = sim->dist_world == 1 && sim->n_parts == 1 && sim->n_streams == 1 && sim->n_stages == 1 && !sim->act_words &&
               sim->max_gread <= 4 * GEM_THREADS && sim->loc_words <= 4096 && !sim->cfg.grid_limit;
  const uint32_t fixed_words = sim->group * (sim->state_words + 4 * GEM_MAX_RAMS_PER_PART + 16) + GEM_MAX_CHUNKS +
                               48 + GEM_WL_CACHE_WORDS + 32 + sim->act_words + (sim->local ? 2 * sim->loc_words : 0u);
  const bool allow_res = !(sim->flags & GEM_F_NO_RESIDENT);
  const uint32_t force_bps = sim->cfg.ctas_per_sm;
  struct Choice { uint32_t bps = 0, grid = 0, area = 0, resident = 0, ring = 0; double score = 0; };
  Choice best;
  std::vector<uint32_t> best_off, off;
  std::vector<uint2> best_items, items;
  double max_cost = 0;
  for (uint32_t p = 0; p < sim->n_parts; p++)
    max_cost = std::max<double>(max_cost, sim->h_parts[(size_t)p * GP_WORDS + GP_COST]);
  for (uint32_t bps = 1; bps <= 4; bps++) {
    if (force_bps && bps != force_bps) continue;
    const int64_t budget = std::min<int64_t>(optin, per_sm / (int64_t)bps - 1024);
    if (budget < (int64_t)(fixed_words * 4 + 2 * slot * 4)) continue;
    const uint32_t area = (uint32_t)(budget / 4) - fixed_words;
    uint32_t grid = std::max<uint32_t>(1, std::min<uint32_t>(sim->max_items, bps * (uint32_t)sms));
    if (grid_limit) grid = std::max<uint32_t>(1, std::min(grid, grid_limit));
    grid = std::min<uint32_t>(grid, GEM_BAR_MAX_CTAS);
    int occ = 0;
    CK(cudaFuncSetAttribute(step_kernel_for(sim), cudaFuncAttributeMaxDynamicSharedMemorySize, (int)budget));
    CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, step_kernel_for(sim), GEM_THREADS, (size_t)budget));
    if ((uint32_t)occ < bps) continue;
    const double makespan = build_worklists(sim, grid, off, items);
    // residency is decided per CTA (its work list's distinct programs fit in the area)
    uint32_t n_res = 0;
    for (uint32_t b = 0; b < grid && allow_res; b++) {
      std::vector<uint32_t> seen;
      uint64_t words = 0;
      bool ok = true;
      for (uint32_t s = 0; s < sim->n_stages && ok; s++)
        for (uint32_t k = off[(size_t)s * (grid + 1) + b]; k < off[(size_t)s * (grid + 1) + b + 1]; k++) {
          const uint32_t p = items[k].x;
          if (std::find(seen.begin(), seen.end(), p) != seen.end()) continue;
          seen.push_back(p);
          words += (sim->h_parts[(size_t)p * GP_WORDS + GP_PROG_LEN] + 3u) & ~3u;
          if (seen.size() > GEM_MAX_RESIDENT || words > area) { ok = false; break; }
        }
      n_res += ok;
    }
    const bool res = n_res == grid;
    uint32_t ring = std::min<uint32_t>(GEM_RING_MAX, area / std::max<uint32_t>(slot, 4));
    ring = ring >= 8 ? 8 : ring >= 4 ? 4 : ring >= 2 ? 2 : ring;   // power of two (kernel masks instead of dividing)
    if (!res && ring < 2) continue;
    // score: estimated makespan, SM sharing slows co-resident CTAs, streaming costs a little
    double score = makespan * (1.0 + 0.5 * (bps - 1) * std::min(1.0, (double)grid / ((double)bps * sms)))
                   * (1.0 + 0.1 * (double)(grid - n_res) / grid);
    if (!best.bps || score < best.score) {
      best.bps = bps; best.grid = grid; best.area = area; best.resident = n_res; best.ring = ring;
      best.score = score;
      best_off.swap(off);
      best_items.swap(items);
    }
  }
  (void)max_cost;
  if (!best.bps) return fail(GEM_E_UNSUPPORTED, "cannot fit the program ring / state in shared memory");
  sim->blocks_per_sm = best.bps;
  sim->grid = best.grid;
  sim->area_words = best.area;
  sim->resident = best.resident;
  sim->ring_slots = best.ring;
  sim->slot_words = slot;
  sim->smem_bytes = (fixed_words + best.area) * 4;
  CK(cudaFuncSetAttribute(step_kernel_for(sim), cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sim->smem_bytes));
  CK(dalloc(&sim->d_wl_off, best_off.size() * 4));
  CK(cudaMemcpy(sim->d_wl_off, best_off.data(), best_off.size() * 4, cudaMemcpyHostToDevice));
  CK(dalloc(&sim->d_wl_items, std::max<size_t>(best_items.size(), 1) * 8));
  if (!best_items.empty())
    CK(cudaMemcpy(sim->d_wl_items, best_items.data(), best_items.size() * 8, cudaMemcpyHostToDevice));
  return GEM_OK;
}

static const void* word_kernel_for(const gem_sim* sim) {
  return sim->local ? (const void*)gem_word_kernel<true> : (const void*)gem_word_kernel<false>;
}

// Word mode launch: one CTA per SM, LPT work lists of (partition, stream)
// items; every distinct program of a CTA's list must fit in its shared memory
// beside the state (else GEM_E_UNSUPPORTED and the bit-packed path runs).
static int plan_launch_words(gem_sim* sim, uint32_t grid_limit) {
  int sms = 0, coop = 0, optin = 0;
  CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, sim->device));
  CK(cudaDeviceGetAttribute(&coop, cudaDevAttrCooperativeLaunch, sim->device));
  CK(cudaDeviceGetAttribute(&optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, sim->device));
  if (!coop) return fail(GEM_E_UNSUPPORTED, "device lacks cooperative launch");
  if (sim->n_stages > GEM_WL_MAX_STAGES) return fail(GEM_E_UNSUPPORTED, "too many stages for word mode");
  sim->sm_count = (uint32_t)sms;
  sim->group = 1;
  sim->max_items = 0;
  for (uint32_t s = 0; s < sim->n_stages; s++)
    sim->max_items = std::max(sim->max_items, (sim->h_stage[s + 1] - sim->h_stage[s]) * sim->n_streams);
  uint32_t grid = std::max<uint32_t>(1, std::min<uint32_t>(sim->max_items, (uint32_t)sms));
  if (grid_limit) grid = std::max<uint32_t>(1, std::min(grid, grid_limit));
  sim->loc_words = sim->q_words_int + sim->n_rams;
  sim->local = grid == 1 && sim->n_streams == 1 && sim->loc_words <= 8192;
  std::vector<uint32_t> off;
  std::vector<uint2> items;
  build_worklists(sim, grid, off, items);
  uint32_t area = 0;
  for (uint32_t b = 0; b < grid; b++) {
    std::vector<uint32_t> seen;
    uint32_t words = 0, n_items = 0;
    for (uint32_t s = 0; s < sim->n_stages; s++)
      for (uint32_t k = off[(size_t)s * (grid + 1) + b]; k < off[(size_t)s * (grid + 1) + b + 1]; k++) {
        n_items++;
        const uint32_t p = items[k].x;
        if (std::find(seen.begin(), seen.end(), p) != seen.end()) continue;
        seen.push_back(p);
        words += sim->h_wprog_len[p];
      }
    if (seen.size() > GEM_MAX_RESIDENT || n_items > GEM_WL_CACHE)
      return fail(GEM_E_UNSUPPORTED, "word mode: too many work items per CTA");
    area = std::max(area, words);
  }
  const uint32_t fixed = sim->word_state + GEM_WORD_RAMP + 3 * 16 + GEM_WL_CACHE_WORDS + 4 + (sim->local ? 2 * sim->loc_words : 0u);
  const uint64_t bytes = (uint64_t)(fixed + area) * 4;
  if (bytes > (uint64_t)optin) return fail(GEM_E_UNSUPPORTED, "word programs do not fit in shared memory");
  CK(cudaFuncSetAttribute(word_kernel_for(sim), cudaFuncAttributeMaxDynamicSharedMemorySize, (int)bytes));
  int occ = 0;
  CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, word_kernel_for(sim), GEM_WORD_THREADS, (size_t)bytes));
  if (occ < 1) return fail(GEM_E_UNSUPPORTED, "word kernel not resident");
  sim->blocks_per_sm = 1;
  sim->grid = grid;
  sim->area_words = area;
  sim->resident = grid;
  sim->ring_slots = 0;
  sim->slot_words = 0;
  sim->smem_bytes = (uint32_t)bytes;
  CK(dalloc(&sim->d_wl_off, off.size() * 4));
  CK(cudaMemcpy(sim->d_wl_off, off.data(), off.size() * 4, cudaMemcpyHostToDevice));
  CK(dalloc(&sim->d_wl_items, std::max<size_t>(items.size(), 1) * 8));
  if (!items.empty()) CK(cudaMemcpy(sim->d_wl_items, items.data(), items.size() * 8, cudaMemcpyHostToDevice));
  return GEM_OK;
}

static const void* lane_kernel_for(uint32_t k, bool v2, uint32_t m) {
  if (v2 && m == 2)
    return k >= 4 ? (const void*)gem_lane_kernel<4, true, 2> : k == 2 ? (const void*)gem_lane_kernel<2, true, 2>
                                                                        : (const void*)gem_lane_kernel<1, true, 2>;
  if (v2)
    return k >= 4 ? (const void*)gem_lane_kernel<4, true, 1> : k == 2 ? (const void*)gem_lane_kernel<2, true, 1>
                                                                        : (const void*)gem_lane_kernel<1, true, 1>;
  return k >= 4 ? (const void*)gem_lane_kernel<4, false, 1> : k == 2 ? (const void*)gem_lane_kernel<2, false, 1>
                                                                       : (const void*)gem_lane_kernel<1, false, 1>;
}

// Lane mode launch: one CTA per SM (all shared memory for the lane state and
// the program ring), work items = (partition, 32-stream group), LPT lists.
static int plan_launch_lanes(gem_sim* sim, uint32_t grid_limit) {
  int sms = 0, coop = 0, optin = 0, per_sm = 0;
  CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, sim->device));
  CK(cudaDeviceGetAttribute(&coop, cudaDevAttrCooperativeLaunch, sim->device));
  CK(cudaDeviceGetAttribute(&optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, sim->device));
  CK(cudaDeviceGetAttribute(&per_sm, cudaDevAttrMaxSharedMemoryPerMultiprocessor, sim->device));
  if (!coop) return fail(GEM_E_UNSUPPORTED, "device lacks cooperative launch");
  sim->sm_count = (uint32_t)sms;
  const uint32_t want_gl = std::min<uint32_t>(sim->cfg.lane_groups ? sim->cfg.lane_groups : 4u, 4u);
  const uint32_t force_bps = sim->cfg.lane_ctas_per_sm;
  // prefer 2 CTAs per SM (16 warps to hide latency), then as many 32-stream
  // groups per work item as fit (shared memory holds only the lane state:
  // records stream from global memory into registers)
  uint32_t bps = 0, gl = 0;
  // (compacted programs: the K <= 2 kernels are built for up to 4 CTAs per SM)
  const uint32_t max_bps = sim->lane_v2 ? 4u : 2u;
  for (uint32_t b = force_bps ? std::min(force_bps, max_bps) : 2u; b >= 1 && !bps; b--) {
    if (force_bps && force_bps != b) continue;
    const uint32_t bud = (uint32_t)std::min<int64_t>(optin, per_sm / (int64_t)b - 1024);
    for (uint32_t k = std::max<uint32_t>(1, std::min(want_gl, sim->n_groups)); k >= 1; k--) {
      if (k == 3) continue;   // the kernel is instantiated for K = 1, 2, 4 interleaved groups
      if (b > 2 && k > 2) continue;   // K = 4 kernels are built for <= 2 CTAs per SM
      const uint64_t words = (uint64_t)k * (sim->lane_words + sim->ramp_words + 16);
      if (words * 4 <= bud) { bps = b; gl = k; break; }
    }
  }
  if (!bps) return fail(GEM_E_UNSUPPORTED, "lane state exceeds shared memory");
  sim->lane_groups = gl;
  sim->group = 32 * gl;    // streams per work item
  sim->max_items = 0;
  for (uint32_t s = 0; s < sim->n_stages; s++)
    sim->max_items = std::max(sim->max_items, (sim->h_stage[s + 1] - sim->h_stage[s]) * ((sim->n_groups + gl - 1) / gl));
  const uint32_t fixed_words = gl * (sim->lane_words + sim->ramp_words + 16);
  uint32_t grid = std::max<uint32_t>(1, std::min<uint32_t>(sim->max_items, bps * (uint32_t)sms));
  if (grid_limit) grid = std::max<uint32_t>(1, std::min(grid, grid_limit));
  grid = std::min<uint32_t>(grid, GEM_BAR_MAX_CTAS);
  const uint32_t smem = fixed_words * 4;
  const void* lk = lane_kernel_for(gl, sim->lane_v2, sim->lane_m);
  CK(cudaFuncSetAttribute(lk, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  int occ = 0;
  CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, lk, GEM_THREADS, smem));
  if ((uint32_t)occ < bps) return fail(GEM_E_UNSUPPORTED, "lane kernel cannot be co-resident");
  std::vector<uint32_t> off;
  std::vector<uint2> items;
  build_worklists(sim, grid, off, items);
  // one stage: dynamic distribution of LPT-ordered units (GEM_F_STATIC_LANES: static lists)
  if (sim->n_stages == 1 && !(sim->flags & GEM_F_STATIC_LANES)) {
    // unit = `run` consecutive items of one partition (they share its records
    // in L2 / L1); as long as there are >= 8 units per CTA
    const uint32_t np1 = sim->h_stage[1] - sim->h_stage[0];
    const uint64_t items1 = (uint64_t)np1 * ((sim->n_streams + sim->group - 1) / sim->group);
    uint32_t run = (uint32_t)std::max<uint64_t>(1, std::min<uint64_t>(4, items1 / (8ull * grid)));
    if (sim->cfg.lane_run) run = sim->cfg.lane_run;
    std::vector<std::pair<double, uint4>> us;
    const uint32_t np = sim->h_stage[1] - sim->h_stage[0];
    for (uint32_t st = 0; st < sim->n_streams; st += sim->group * run)
      for (uint32_t k = 0; k < np; k++) {
        const uint32_t p = sim->h_stage[sim->n_stages + 1 + k];
        const uint32_t n_items = std::min(run, (sim->n_streams - st + sim->group - 1) / sim->group);
        us.push_back({(double)sim->h_parts[(size_t)p * GP_WORDS + GP_COST] * n_items, make_uint4(p, st, n_items, 0)});
      }
    std::stable_sort(us.begin(), us.end(), [](const std::pair<double, uint4>& x, const std::pair<double, uint4>& y) {
      return x.first > y.first;
    });
    std::vector<uint4> hu;
    for (auto& u : us) hu.push_back(u.second);
    sim->n_units = (uint32_t)hu.size();
    CK(dalloc(&sim->d_dyn_units, hu.size() * 16));
    CK(cudaMemcpy(sim->d_dyn_units, hu.data(), hu.size() * 16, cudaMemcpyHostToDevice));
    CK(dalloc(&sim->d_dyn_ctr, 16));
    grid = std::min<uint32_t>(grid, sim->n_units);
  }
  sim->blocks_per_sm = bps;
  sim->grid = grid;
  sim->area_words = 0;
  sim->ring_slots = 0;
  sim->slot_words = 0;
  sim->resident = 0;
  sim->smem_bytes = smem;
  CK(dalloc(&sim->d_wl_off, off.size() * 4));
  CK(cudaMemcpy(sim->d_wl_off, off.data(), off.size() * 4, cudaMemcpyHostToDevice));
  CK(dalloc(&sim->d_wl_items, std::max<size_t>(items.size(), 1) * 8));
  if (!items.empty()) CK(cudaMemcpy(sim->d_wl_items, items.data(), items.size() * 8, cudaMemcpyHostToDevice));
  return GEM_OK;
}

extern "C" {

const char* gem_last_error(void) { return g_err.c_str(); }

}  // extern "C"

// Structural validation of a program blob (include/gem.h: a malformed or
// truncated blob is GEM_E_FORMAT, never an out-of-bounds access): every table
// offset + length inside the blob, permutation entries in range, stage prefix
// monotone, every partition program inside the program area with a sane
// header and chunk table (at most GEM_MAX_CHUNKS chunks: the kernel keeps the
// chunk table in a fixed shared-memory array).
static int validate_blob(const uint32_t* w, size_t nw) {
  auto in = [&](uint64_t off, uint64_t len) { return off <= nw && len <= nw - off; };
  const uint64_t prog_words = w[GH_PROG_WORDS_LO] | ((uint64_t)w[GH_PROG_WORDS_HI] << 32);
  const uint32_t n_parts = w[GH_N_PARTS], n_stages = w[GH_N_STAGES];
  if (!in(w[GH_OFF_PROG], prog_words)) return fail(GEM_E_FORMAT, "truncated program area");
  if (n_stages == 0 || n_stages > GEM_WL_MAX_STAGES) return fail(GEM_E_FORMAT, "bad stage count");
  if (!in(w[GH_OFF_PARTS], (uint64_t)n_parts * GP_WORDS)) return fail(GEM_E_FORMAT, "truncated partition table");
  if (!in(w[GH_OFF_STAGES], (uint64_t)n_stages + 1 + n_parts)) return fail(GEM_E_FORMAT, "truncated stage list");
  const uint32_t* st = w + w[GH_OFF_STAGES];
  if (st[0] != 0 || st[n_stages] > n_parts) return fail(GEM_E_FORMAT, "bad stage prefix");
  for (uint32_t s = 0; s < n_stages; s++)
    if (st[s + 1] < st[s]) return fail(GEM_E_FORMAT, "stage prefix not monotone");
  for (uint32_t k = 0; k < st[n_stages]; k++)
    if (st[n_stages + 1 + k] >= n_parts) return fail(GEM_E_FORMAT, "bad partition id in stage list");
  const uint64_t qw = w[GH_Q_WORDS], pw = w[GH_PO_WORDS];
  if (qw * 32 < w[GH_N_FLOPS] || pw * 32 < w[GH_N_PO] || (uint64_t)w[GH_PI_WORDS] * 32 < w[GH_N_PI])
    return fail(GEM_E_FORMAT, "word counts too small");
  if (!in(w[GH_OFF_FLOP_INIT], qw + qw * 32 + pw * 32)) return fail(GEM_E_FORMAT, "truncated permutation tables");
  const uint32_t* q_ext = w + w[GH_OFF_FLOP_INIT] + qw;
  const uint32_t* po_ext = q_ext + qw * 32;
  for (uint64_t b = 0; b < qw * 32; b++)
    if (q_ext[b] != 0xFFFFFFFFu && q_ext[b] >= w[GH_N_FLOPS]) return fail(GEM_E_FORMAT, "bad flop permutation");
  for (uint64_t b = 0; b < pw * 32; b++)
    if (po_ext[b] != 0xFFFFFFFFu && po_ext[b] >= w[GH_N_PO]) return fail(GEM_E_FORMAT, "bad PO permutation");
  const uint32_t* parts = w + w[GH_OFF_PARTS];
  const uint32_t* prog = w + w[GH_OFF_PROG];
  const uint64_t lp_words = w[GH_LANE_PROG_WORDS_LO] | ((uint64_t)w[GH_LANE_PROG_WORDS_HI] << 32);
  if (w[GH_HAS_LANES] && !in(w[GH_OFF_LANE_PROG], lp_words)) return fail(GEM_E_FORMAT, "truncated lane programs");
  for (uint32_t p = 0; p < n_parts; p++) {
    const uint32_t* e = parts + (size_t)p * GP_WORDS;
    const uint64_t off = e[GP_PROG_OFF], len = e[GP_PROG_LEN];
    if (off + len > prog_words || len < PH_WORDS) return fail(GEM_E_FORMAT, "partition program out of range");
    const uint32_t* pr = prog + off;
    if (pr[PH_MAGIC] != GEM_PART_MAGIC || pr[PH_N_RAM] > GEM_MAX_RAMS_PER_PART || pr[PH_N_LAYERS] != e[GP_N_LAYERS])
      return fail(GEM_E_FORMAT, "bad partition program header");
    if (pr[PH_N_CHUNKS] != pr[PH_N_LAYERS] + 2)
      return fail(GEM_E_FORMAT, "bad chunk count");
    if (pr[PH_N_CHUNKS] > GEM_MAX_CHUNKS)
      return fail(GEM_E_UNSUPPORTED, "partition program has more than " + std::to_string(GEM_MAX_CHUNKS - 2) +
                                         " layers (map with a smaller part_size)");
    if ((uint64_t)pr[PH_OFF_CHUNKS] + pr[PH_N_CHUNKS] > len) return fail(GEM_E_FORMAT, "bad chunk table");
    uint64_t sum = 0, mx = 0;
    for (uint32_t k = 0; k < pr[PH_N_CHUNKS]; k++) {
      const uint32_t c = pr[pr[PH_OFF_CHUNKS] + k];
      if (c & 3u) return fail(GEM_E_FORMAT, "chunk not a multiple of 16 bytes");
      sum += c;
      mx = std::max<uint64_t>(mx, c);
    }
    if (sum > len || mx > w[GH_MAX_CHUNK_WORDS]) return fail(GEM_E_FORMAT, "chunk table exceeds program");
    if (e[GP_CHUNK0] != pr[pr[PH_OFF_CHUNKS]]) return fail(GEM_E_FORMAT, "partition table / chunk table mismatch");
    if (pr[PH_OFF_GREAD] + 2ull * pr[PH_N_GREAD] > len || pr[PH_OFF_OUT] + pr[PH_N_OUT_PAD] + 32ull * pr[PH_N_OUT] > len)
      return fail(GEM_E_FORMAT, "partition sections out of range");
    if (w[GH_HAS_LANES] && (uint64_t)e[GP_LANE_OFF] + e[GP_LANE_LEN] > lp_words)
      return fail(GEM_E_FORMAT, "lane program out of range");
  }
  if (w[GH_HAS_WORDS]) {
    // word programs (WRD1): every table inside its program, every op / output
    // byte offset inside the state, every port and output gid inside its region
    const uint64_t wp_words = w[GH_WORD_PROG_WORDS_LO] | ((uint64_t)w[GH_WORD_PROG_WORDS_HI] << 32);
    if (!in(w[GH_OFF_WORD_PROG], wp_words) || (w[GH_OFF_WORD_PROG] & 3u)) return fail(GEM_E_FORMAT, "truncated word programs");
    const uint32_t* wp = w + w[GH_OFF_WORD_PROG];
    for (uint32_t p = 0; p < n_parts; p++) {
      const uint64_t off = parts[(size_t)p * GP_WORDS + GP_WORD_OFF];
      if ((off & 3u) || off + WPH_WORDS > wp_words) return fail(GEM_E_FORMAT, "word program out of range");
      const uint32_t* h = wp + off;
      const uint64_t len = h[WPH_PROG_LEN], sw = h[WPH_STATE_WORDS];
      if (h[WPH_MAGIC] != GEM_WORD_MAGIC || len < WPH_WORDS || (len & 3u) || off + len > wp_words || len > w[GH_WORD_MAX_PROG] ||
          sw > GEM_WORD_MAX_WORDS || sw > w[GH_WORD_MAX_STATE] || sw < 1 + (uint64_t)h[WPH_N_GREAD] ||
          h[WPH_N_RAM] > GEM_MAX_RAMS_PER_PART)
        return fail(GEM_E_FORMAT, "bad word program header");
      const uint64_t ns = h[WPH_N_STEPS], no = h[WPH_N_OPS], nout = h[WPH_N_OUT], nr = h[WPH_N_RAM], ng = h[WPH_N_GREAD];
      if (h[WPH_OFF_STEPS] + ns + 1 > len || (h[WPH_OFF_OPS] & 1u) || h[WPH_OFF_OPS] + 2 * no > len ||
          h[WPH_OFF_OUT] + 33 * nout > len || h[WPH_OFF_RAM] + 4 * nr > len || h[WPH_OFF_GREAD] + ng > len)
        return fail(GEM_E_FORMAT, "word program sections out of range");
      const uint32_t* stp = h + h[WPH_OFF_STEPS];
      if (stp[0] != 0 || stp[ns] != no) return fail(GEM_E_FORMAT, "bad word step table");
      for (uint64_t k = 0; k < ns; k++)
        if (stp[k + 1] < stp[k] || stp[k + 1] - stp[k] > 4u * GEM_THREADS)
          return fail(GEM_E_FORMAT, "word step table not monotone or a step above 1024 ops");
      const uint32_t lim = (uint32_t)sw * 4;
      const uint32_t* ops = h + h[WPH_OFF_OPS];
      for (uint64_t i = 0; i < no; i++) {
        const uint32_t x = ops[2 * i], y = ops[2 * i + 1];
        if ((x & 0xFFFCu) >= lim || ((x >> 16) & 0xFFFCu) >= lim || y >= lim || y == 0 || (y & 3u))
          return fail(GEM_E_FORMAT, "word op outside the state");
      }
      const uint32_t* od = h + h[WPH_OFF_OUT];
      for (uint64_t o = 0; o < nout; o++) {
        const uint32_t reg = GEM_GID_REGION(od[o]), idx = GEM_GID_INDEX(od[o]);
        const bool ok = (reg == GEM_R_Q && idx < qw) || (reg == GEM_R_PO && idx < pw) ||
                        (reg == GEM_R_CUT && idx < w[GH_CUT_WORDS]) || (reg == GEM_R_RAMP && idx < 4 * nr);
        if (!ok) return fail(GEM_E_FORMAT, "bad word output gid");
        for (uint32_t k = 0; k < 32; k++)
          if ((od[nout + o * 32 + k] & 0xFFFCu) >= lim || (od[nout + o * 32 + k] >> 16))
            return fail(GEM_E_FORMAT, "word output outside the state");
      }
      const uint32_t* rr = h + h[WPH_OFF_RAM];
      for (uint64_t r = 0; r < nr; r++)
        if (rr[4 * r] >= w[GH_N_RAMS]) return fail(GEM_E_FORMAT, "bad word RAM id");
      const uint32_t* gr = h + h[WPH_OFF_GREAD];
      for (uint64_t k = 0; k < ng; k++) {
        const uint32_t reg = gr[k] >> 24, bit = gr[k] & 0xFFFFFFu;
        const bool ok = (reg == GEM_R_PI && bit < 32ull * w[GH_PI_WORDS]) || (reg == GEM_R_Q && bit < 32 * qw) ||
                        (reg == GEM_R_RD && bit < 32ull * w[GH_N_RAMS]) || (reg == GEM_R_CUT && bit < 32ull * w[GH_CUT_WORDS]);
        if (!ok) return fail(GEM_E_FORMAT, "bad word port gid");
      }
    }
  }
  return GEM_OK;
}

// gem_load_program body; on failure the caller frees the partially built handle.
// Partition -> rank split of a design over `world` devices (gem_dist_owner):
// per stage (stages are separated by barriers, so each is balanced on its
// own), partitions in decreasing mapper cost go to the least-loaded rank
// (ties: the rank with less work over the earlier stages, then the lower rank).
static void dist_assign(const uint32_t* parts, const uint32_t* stages, uint32_t n_stages, uint32_t world,
                        uint32_t* owner) {
  std::vector<uint64_t> total(world, 0);
  for (uint32_t s = 0; s < n_stages; s++) {
    std::vector<std::pair<uint32_t, uint32_t>> ps;   // (cost, partition)
    for (uint32_t k = stages[s]; k < stages[s + 1]; k++) {
      const uint32_t p = stages[n_stages + 1 + k];
      ps.push_back({parts[(size_t)p * GP_WORDS + GP_COST], p});
    }
    std::stable_sort(ps.begin(), ps.end(), [](const std::pair<uint32_t, uint32_t>& a,
                                              const std::pair<uint32_t, uint32_t>& b) { return a.first > b.first; });
    std::vector<uint64_t> load(world, 0);
    for (auto& x : ps) {
      uint32_t r = 0;
      for (uint32_t q = 1; q < world; q++)
        if (load[q] < load[r] || (load[q] == load[r] && total[q] < total[r])) r = q;
      owner[x.second] = r;
      load[r] += std::max<uint32_t>(x.first, 1);
    }
    for (uint32_t q = 0; q < world; q++) total[q] += load[q];
  }
}

static int load_impl(gem_sim* sim, const uint32_t* w, size_t nw, const gem_config* cfg) {
  sim->device = cfg->device;
  sim->cfg = *cfg;
  sim->flags = cfg->flags;
  sim->n_streams = cfg->n_streams;
  sim->dist_world = std::max<uint32_t>(1, cfg->dist_world);
  sim->dist_rank = cfg->dist_rank;
  if (sim->dist_world > 1) sim->flags &= ~GEM_F_ACTIVITY;   // the DIST kernel has no pruning build
  CK(cudaSetDevice(sim->device));
  const uint64_t prog_words = w[GH_PROG_WORDS_LO] | ((uint64_t)w[GH_PROG_WORDS_HI] << 32);
  sim->n_pi = w[GH_N_PI]; sim->n_po = w[GH_N_PO]; sim->n_flops = w[GH_N_FLOPS]; sim->n_rams = w[GH_N_RAMS];
  sim->n_parts = w[GH_N_PARTS]; sim->n_stages = w[GH_N_STAGES]; sim->max_layers = w[GH_MAX_LAYERS];
  sim->total_layers = w[GH_TOTAL_LAYERS];
  sim->state_words = std::max<uint32_t>(w[GH_MAX_STATE_WORDS], 32);
  sim->state_words = (sim->state_words + 3) & ~3u;
  sim->pi_words = w[GH_PI_WORDS]; sim->po_words_int = w[GH_PO_WORDS]; sim->q_words_int = w[GH_Q_WORDS];
  sim->cut_words = w[GH_CUT_WORDS];
  sim->po_words_ext = (sim->n_po + 31) / 32;
  sim->q_words_ext = (sim->n_flops + 31) / 32;
  sim->n_and = w[GH_N_AND_LO] | ((uint64_t)w[GH_N_AND_HI] << 32);
  sim->n_and_mapped = w[GH_N_AND_MAPPED_LO] | ((uint64_t)w[GH_N_AND_MAPPED_HI] << 32);
  sim->program_bytes = prog_words * 4;
  const uint32_t* parts = w + w[GH_OFF_PARTS];
  const uint32_t* stages = w + w[GH_OFF_STAGES];
  const uint32_t* finit = w + w[GH_OFF_FLOP_INIT];
  const uint32_t* q_ext_of_int = finit + sim->q_words_int;
  const uint32_t* po_ext_of_int = q_ext_of_int + (size_t)sim->q_words_int * 32;
  for (uint32_t s = 0; s < sim->n_stages; s++)
    sim->max_items = std::max(sim->max_items, (stages[s + 1] - stages[s]) * sim->n_streams);
  for (uint32_t p = 0; p < sim->n_parts; p++) {
    const uint32_t* pr = w + w[GH_OFF_PROG] + parts[p * GP_WORDS + GP_PROG_OFF];
    if (sim->flags & GEM_F_ACTIVITY) sim->act_words = std::max(sim->act_words, (pr[PH_N_GREAD] + 3u) & ~3u);
    sim->max_gread = std::max(sim->max_gread, pr[PH_N_GREAD]);
  }
  // inverse permutation tables
  std::vector<uint32_t> q_int_of_ext(std::max<uint32_t>(sim->n_flops, 1), 0),
      po_int_of_ext(std::max<uint32_t>(sim->n_po, 1), 0);
  for (uint32_t b = 0; b < sim->q_words_int * 32; b++)
    if (q_ext_of_int[b] != 0xFFFFFFFFu) q_int_of_ext[q_ext_of_int[b]] = b;
  for (uint32_t b = 0; b < sim->po_words_int * 32; b++)
    if (po_ext_of_int[b] != 0xFFFFFFFFu) po_int_of_ext[po_ext_of_int[b]] = b;
  // streams / events / watchdog words (mapped pinned host memory)
  if (cfg->cuda_stream) sim->stream = (cudaStream_t)cfg->cuda_stream;
  else { CK(cudaStreamCreateWithFlags(&sim->stream, cudaStreamNonBlocking)); sim->own_stream = true; }
  CK(cudaEventCreate(&sim->ev0));
  CK(cudaEventCreate(&sim->ev1));
  CK(cudaEventCreateWithFlags(&sim->ev_in, cudaEventDisableTiming));
  CK(cudaHostAlloc((void**)&sim->h_err, 64, cudaHostAllocMapped));
  std::memset(sim->h_err, 0, 64);
  CK(cudaHostGetDevicePointer((void**)&sim->d_err, sim->h_err, 0));
  // lane mode: >= 32 streams and lane programs present (GEM_F_NO_LANES disables)
  sim->lanes = (w[GH_HAS_LANES] && cfg->n_streams >= 32 && !(cfg->flags & GEM_F_NO_LANES) && sim->dist_world == 1)
                   ? 1u : 0u;
  if (sim->lanes) {
    sim->n_groups = (cfg->n_streams + 31) / 32;
    sim->lane_words = (std::max<uint32_t>(w[GH_LANE_MAX_WORDS], 4) + 3) & ~3u;
    sim->lane_max_chunk = w[GH_LANE_MAX_CHUNK_WORDS];
    sim->ramp_words = std::max<uint32_t>(w[GH_MAX_RAMS_PART], 1) * 128;
    const uint32_t* lp = w + w[GH_OFF_LANE_PROG];
    sim->lane_v2 = sim->n_parts && lp[parts[GP_LANE_OFF] + LPH_MAGIC] == GEM_LANE2_MAGIC;
    sim->lane_m = sim->lane_v2 ? std::max<uint32_t>(1, lp[parts[GP_LANE_OFF] + LPH_OPS_PER_THREAD]) : 1u;
    for (uint32_t p = 0; p < sim->n_parts; p++) {
      const uint32_t* h = lp + parts[(size_t)p * GP_WORDS + GP_LANE_OFF];
      if (h[LPH_MAGIC] != (sim->lane_v2 ? GEM_LANE2_MAGIC : GEM_LANE_MAGIC) ||
          (sim->lane_v2 && std::max<uint32_t>(1, h[LPH_OPS_PER_THREAD]) != sim->lane_m) || sim->lane_m > 2)
        return fail(GEM_E_FORMAT, "mixed or bad lane programs");
    }
  }
  // word mode: single-stream latency path (GEM_F_NO_WORDS, activity pruning
  // and split designs keep the bit-packed path); planned below, falls back to
  // the bit-packed path when the programs do not fit in shared memory
  sim->words = !sim->lanes && w[GH_HAS_WORDS] && sim->dist_world == 1 &&
               !(sim->flags & (GEM_F_NO_WORDS | GEM_F_ACTIVITY));
  if (sim->words) {
    const uint64_t wp_words = w[GH_WORD_PROG_WORDS_LO] | ((uint64_t)w[GH_WORD_PROG_WORDS_HI] << 32);
    sim->word_state = (std::max<uint32_t>(w[GH_WORD_MAX_STATE], 4) + 3) & ~3u;
    CK(dalloc(&sim->d_wprog, wp_words * 4));
    CK(cudaMemcpy(sim->d_wprog, w + w[GH_OFF_WORD_PROG], wp_words * 4, cudaMemcpyHostToDevice));
    sim->h_wprog_len.resize(sim->n_parts);
    for (uint32_t p = 0; p < sim->n_parts; p++)
      sim->h_wprog_len[p] = w[w[GH_OFF_WORD_PROG] + parts[(size_t)p * GP_WORDS + GP_WORD_OFF] + WPH_PROG_LEN];
  }
  // uploads
  const size_t S = sim->n_streams;
  CK(dalloc(&sim->d_prog, prog_words * 4));
  CK(cudaMemcpy(sim->d_prog, w + w[GH_OFF_PROG], prog_words * 4, cudaMemcpyHostToDevice));
  CK(dalloc(&sim->d_parts, (size_t)sim->n_parts * GP_WORDS * 4));
  CK(cudaMemcpy(sim->d_parts, parts, (size_t)sim->n_parts * GP_WORDS * 4, cudaMemcpyHostToDevice));
  const size_t stage_words = sim->n_stages + 1 + sim->n_parts;
  CK(dalloc(&sim->d_stage, stage_words * 4));
  CK(cudaMemcpy(sim->d_stage, stages, stage_words * 4, cudaMemcpyHostToDevice));
  CK(dalloc(&sim->d_q_int_of_ext, q_int_of_ext.size() * 4));
  CK(cudaMemcpy(sim->d_q_int_of_ext, q_int_of_ext.data(), q_int_of_ext.size() * 4, cudaMemcpyHostToDevice));
  CK(dalloc(&sim->d_q_ext_of_int, (size_t)sim->q_words_int * 32 * 4));
  CK(cudaMemcpy(sim->d_q_ext_of_int, q_ext_of_int, (size_t)sim->q_words_int * 32 * 4, cudaMemcpyHostToDevice));
  CK(dalloc(&sim->d_po_int_of_ext, po_int_of_ext.size() * 4));
  CK(cudaMemcpy(sim->d_po_int_of_ext, po_int_of_ext.data(), po_int_of_ext.size() * 4, cudaMemcpyHostToDevice));
  if (sim->lanes) {
    const uint64_t lp_words = w[GH_LANE_PROG_WORDS_LO] | ((uint64_t)w[GH_LANE_PROG_WORDS_HI] << 32);
    CK(dalloc(&sim->d_lprog, lp_words * 4));
    CK(cudaMemcpy(sim->d_lprog, w + w[GH_OFF_LANE_PROG], lp_words * 4, cudaMemcpyHostToDevice));
    const size_t G = sim->n_groups, qb = (size_t)sim->q_words_int * 32;
    CK(dalloc(&sim->d_q, 2 * qb * G * 4));
    CK(dalloc(&sim->d_rd, 2 * (size_t)std::max<uint32_t>(sim->n_rams, 1) * 32 * G * 4));
    CK(dalloc(&sim->d_cut, (size_t)std::max<uint32_t>(sim->cut_words, 1) * 32 * G * 4));
  } else {
    CK(dalloc(&sim->d_q, 2 * S * sim->q_words_int * 4));
    CK(dalloc(&sim->d_rd, 2 * S * std::max<uint32_t>(sim->n_rams, 1) * 4));
    CK(dalloc(&sim->d_cut, S * std::max<uint32_t>(sim->cut_words, 1) * 4));
  }
  CK(dalloc(&sim->d_mem, S * sim->n_rams * (size_t)GEM_RAM_WORDS * 4));
  CK(dalloc(&sim->d_bar, (size_t)(GEM_BAR_MAX_CTAS + 2) * GEM_BAR_STRIDE * 8));
  CK(dalloc(&sim->d_act, 16));
  CK(cudaMemset(sim->d_act, 0, 16));
  // initial state: flops = init (U5), RD = 0, RAM = 0 (U10)
  if (sim->lanes) {
    const size_t G = sim->n_groups, qb = (size_t)sim->q_words_int * 32;
    std::vector<uint32_t> q0(2 * qb * G, 0);
    for (size_t b = 0; b < qb; b++)
      if ((finit[b / 32] >> (b % 32)) & 1u)
        for (size_t g = 0; g < G; g++) q0[b * G + g] = 0xFFFFFFFFu;   // X[buf 0][bit][group]
    CK(cudaMemcpy(sim->d_q, q0.data(), q0.size() * 4, cudaMemcpyHostToDevice));
    CK(cudaMemset(sim->d_rd, 0, 2 * (size_t)std::max<uint32_t>(sim->n_rams, 1) * 32 * G * 4));
    CK(cudaMemset(sim->d_cut, 0, (size_t)std::max<uint32_t>(sim->cut_words, 1) * 32 * G * 4));
  } else {
    std::vector<uint32_t> q0(S * sim->q_words_int);
    for (size_t s = 0; s < S; s++) std::memcpy(&q0[s * sim->q_words_int], finit, sim->q_words_int * 4);
    CK(cudaMemcpy(sim->d_q, q0.data(), q0.size() * 4, cudaMemcpyHostToDevice));
    CK(cudaMemset(sim->d_q + S * sim->q_words_int, 0, S * sim->q_words_int * 4));
    CK(cudaMemset(sim->d_rd, 0, 2 * S * std::max<uint32_t>(sim->n_rams, 1) * 4));
    CK(cudaMemset(sim->d_cut, 0, S * std::max<uint32_t>(sim->cut_words, 1) * 4));
  }
  if (sim->n_rams) CK(cudaMemset(sim->d_mem, 0, S * sim->n_rams * (size_t)GEM_RAM_WORDS * 4));
  // persistent co-resident grid + shared-memory program placement
  sim->h_parts.assign(parts, parts + (size_t)sim->n_parts * GP_WORDS);
  sim->h_stage.assign(stages, stages + stage_words);
  if (sim->dist_world > 1) {
    sim->owner.assign(sim->n_parts, 0);
    dist_assign(parts, stages, sim->n_stages, sim->dist_world, sim->owner.data());
  }
  if (sim->words && plan_launch_words(sim, cfg->grid_limit) != GEM_OK) {
    if (sim->poisoned) return GEM_E_CUDA;
    sim->words = false;   // does not fit: the bit-packed path runs it
  }
  if (sim->lanes) {
    if (int r = plan_launch_lanes(sim, cfg->grid_limit)) return r;
  } else if (!sim->words) {
    if (int r = plan_launch(sim, w[GH_MAX_CHUNK_WORDS], cfg->grid_limit)) return r;
  }
  CK(cudaDeviceSynchronize());
  return GEM_OK;
}

extern "C" {

int gem_load_program(const void* blob, size_t nbytes, const gem_config* cfg, gem_sim** out) {
  if (!blob || !cfg || !out || nbytes < GH_N_WORDS * 4 || (nbytes & 3)) return fail(GEM_E_INVAL, "bad arguments");
  *out = nullptr;
  const uint32_t* w = (const uint32_t*)blob;
  const size_t nw = nbytes / 4;
  if (w[GH_MAGIC] != GEM_MAGIC || w[GH_VERSION] != GEM_VERSION) return fail(GEM_E_FORMAT, "bad blob magic/version");
  const uint64_t total_words = w[GH_TOTAL_WORDS_LO] | ((uint64_t)w[GH_TOTAL_WORDS_HI] << 32);
  if (total_words != nw) return fail(GEM_E_FORMAT, "truncated blob");
  if (cfg->n_streams == 0) return fail(GEM_E_INVAL, "n_streams must be >= 1");
  if (cfg->dist_world > GEM_DIST_MAX || (cfg->dist_world > 1 && cfg->dist_rank >= cfg->dist_world))
    return fail(GEM_E_INVAL, "bad dist_world / dist_rank");
  if (w[GH_MAX_STATE_WORDS] > GEM_MAX_STATE_WORDS) return fail(GEM_E_FORMAT, "state too large");
  if (int r = validate_blob(w, nw)) return r;
  int ndev = 0;
  if (cudaGetDeviceCount(&ndev) != cudaSuccess || ndev == 0)
    return fail(GEM_E_UNSUPPORTED, "no CUDA device (libgem has no CPU fallback)");
  if (cfg->device < 0 || cfg->device >= ndev) return fail(GEM_E_INVAL, "bad device ordinal");
  gem_sim* sim = new gem_sim();
  if (int r = load_impl(sim, w, nw, cfg)) {
    const std::string msg = g_err;   // gem_free must not clobber the reason
    gem_free(sim);
    g_err = msg;
    return r;
  }
  *out = sim;
  return GEM_OK;
}

int gem_info_get(const gem_sim* sim, gem_info* out) {
  if (!sim || !out) return fail(GEM_E_INVAL, "null argument");
  out->n_pi = sim->n_pi; out->n_po = sim->n_po; out->n_flops = sim->n_flops; out->n_rams = sim->n_rams;
  out->n_parts = sim->n_parts; out->n_stages = sim->n_stages; out->max_layers = sim->max_layers;
  out->total_layers = sim->total_layers;
  out->pi_words = sim->pi_words; out->po_words = sim->po_words_ext; out->q_words = sim->q_words_ext;
  out->grid = sim->grid; out->blocks_per_sm = sim->blocks_per_sm; out->smem_bytes = sim->smem_bytes;
  out->resident = sim->resident; out->ring_slots = sim->ring_slots; out->group = sim->group;
  out->lanes = sim->lanes;
  out->words = sim->words ? 1u : 0u;
  out->n_streams = sim->n_streams;
  out->n_and = sim->n_and; out->n_and_mapped = sim->n_and_mapped; out->program_bytes = sim->program_bytes;
  out->cycle = sim->cycle;
  return GEM_OK;
}

int gem_set_inputs(gem_sim* sim, const uint32_t* pi, uint64_t ncycles, int src_on_device) {
  if (int r = check(sim)) return r;
  if (!pi && ncycles) return fail(GEM_E_INVAL, "null input");
  if (ncycles > 0xFFFFFFF0ull) return fail(GEM_E_INVAL, "too many cycles");
  CK(cudaSetDevice(sim->device));
  if (sim->in_cap < ncycles || !sim->d_pi) {
    if (sim->d_pi) cudaFree(sim->d_pi);
    sim->d_pi = nullptr;
    sim->in_cap = 0;
    uint32_t cap = std::max<uint32_t>((uint32_t)ncycles, 16);
    CK(dalloc(&sim->d_pi, (size_t)sim->n_streams * cap * std::max<uint32_t>(sim->pi_words, 1) * 4));
    if (sim->lanes) {
      if (sim->d_pi_lane) cudaFree(sim->d_pi_lane);
      sim->d_pi_lane = nullptr;
      CK(dalloc(&sim->d_pi_lane, (size_t)cap * std::max<uint32_t>(sim->pi_words, 1) * 32 * sim->n_groups * 4));
    }
    sim->in_cap = cap;
  }
  if (ncycles && sim->pi_words) {
    const size_t row = (size_t)ncycles * sim->pi_words * 4;
    CK(cudaMemcpy2DAsync(sim->d_pi, (size_t)sim->in_cap * sim->pi_words * 4, pi, row, row, sim->n_streams,
                         src_on_device ? cudaMemcpyDeviceToDevice : cudaMemcpyHostToDevice, sim->stream));
    if (sim->lanes) {
      const uint64_t warps = ncycles * sim->n_groups * sim->pi_words;
      to_lanes_kernel<<<(unsigned)std::min<uint64_t>(65535, (warps * 32 + 255) / 256), 256, 0, sim->stream>>>(
          sim->d_pi, sim->d_pi_lane, sim->n_streams, (uint32_t)ncycles, sim->pi_words,
          (uint64_t)sim->in_cap * sim->pi_words, sim->pi_words, sim->n_groups, 0);
      CK(cudaGetLastError());
    }
    if (!src_on_device) {
      // the caller may reuse its (possibly pinned) buffer as soon as we return
      CK(cudaEventRecord(sim->ev_in, sim->stream));
      CK(cudaEventSynchronize(sim->ev_in));
    }
  }
  sim->in_queued = (uint32_t)ncycles;
  sim->in_head = 0;
  return GEM_OK;
}

int gem_step(gem_sim* sim, uint64_t ncycles) {
  if (int r = check(sim)) return r;
  if (ncycles == 0) return GEM_OK;
  if (ncycles > (uint64_t)(sim->in_queued - sim->in_head))
    return fail(GEM_E_NOINPUT, "gem_step: not enough queued input cycles");
  CK(cudaSetDevice(sim->device));
  if (sim->dist_world > 1 && !sim->dist_connected) return fail(GEM_E_INVAL, "dist handle: gem_dist_connect first");
  if (int r = ensure_out(sim, (uint32_t)ncycles)) return r;
  KParams kp;
  std::memset(&kp, 0, sizeof(kp));
  kp.prog = sim->d_prog; kp.parts = sim->d_parts; kp.stage_list = sim->d_stage;
  kp.pi = sim->d_pi; kp.po = sim->d_po; kp.q = sim->d_q; kp.rd = sim->d_rd; kp.cut = sim->d_cut;
  kp.mem = sim->d_mem; kp.q_trace = sim->d_qtrace; kp.digest = sim->d_digest;
  kp.q_int_of_ext = sim->d_q_int_of_ext; kp.bar = sim->d_bar; kp.err = sim->d_err;
  kp.t0 = sim->cycle; kp.ncycles = (uint32_t)ncycles; kp.in_base = sim->in_head; kp.in_cap = sim->in_cap;
  kp.out_cap = sim->out_cap; kp.n_stages = sim->n_stages; kp.n_streams = sim->n_streams;
  kp.state_words = sim->state_words; kp.pi_words = sim->pi_words; kp.po_words = sim->po_words_int;
  kp.q_words = sim->q_words_int; kp.cut_words = sim->cut_words; kp.n_rams = sim->n_rams;
  kp.n_flops = sim->n_flops; kp.q_ext_words = sim->q_words_ext;
  kp.flags = sim->flags & (GEM_F_TRACE_STATE | GEM_F_DIGEST);
  kp.area_words = sim->area_words; kp.slot_words = sim->slot_words; kp.ring_slots = sim->ring_slots;
  kp.allow_resident = sim->resident ? 1u : 0u;   // per-CTA decision in the kernel
  kp.wl_off = sim->d_wl_off;
  kp.group = sim->group;
  kp.wl_items = sim->d_wl_items;
  kp.act_cnt = sim->d_act;
  {
    // programs larger than half the L2 (C4): keep a fraction L2-resident
    // (gem_config::l2_evict_last: 0 = this rule, > 0 = that fraction, < 0 = none)
    int l2 = 0;
    cudaDeviceGetAttribute(&l2, cudaDevAttrL2CacheSize, sim->device);
    float f = 0.f;
    if (!sim->lanes && 2 * sim->program_bytes > (uint64_t)l2)   // does not stay resident by itself
      f = std::min(0.9f, 0.6f * (float)l2 / (float)sim->program_bytes);
    if (sim->cfg.l2_evict_last != 0.f) f = sim->cfg.l2_evict_last;
    kp.l2_frac = std::max(0.f, std::min(1.f, f));
  }
  kp.dyn_units = sim->d_dyn_units;
  kp.n_units = sim->n_units;
  kp.dyn_ctr = sim->d_dyn_ctr;
  if (sim->d_dyn_ctr) CK(cudaMemsetAsync(sim->d_dyn_ctr, 0, 16, sim->stream));
  kp.act_words = sim->lanes ? 0u : sim->act_words;
  kp.loc_words = sim->local ? sim->loc_words : 0u;
  if (sim->dist_world > 1) {
    kp.dist_world = sim->dist_world;
    kp.dist_rank = sim->dist_rank;
    kp.dist_epoch0 = sim->dist_epoch;
    kp.dist_flags = sim->d_dist_flags;
    kp.dist_slots = 0;
    for (uint32_t r = 0; r < sim->dist_world; r++) {
      kp.dist_grid[r] = sim->peers[r].grid;
      kp.dist_slots += sim->peers[r].grid;
      if (r == sim->dist_rank) continue;   // (dist_put skips the own rank)
      kp.peer_q[r] = (uint32_t*)sim->peers[r].q;
      kp.peer_rd[r] = (uint32_t*)sim->peers[r].rd;
      kp.peer_cut[r] = (uint32_t*)sim->peers[r].cut;
      kp.peer_po[r] = (uint32_t*)sim->peers[r].po;
    }
    for (uint32_t r = 0; r < sim->dist_world; r++) kp.peer_flags[r] = (unsigned long long*)sim->peers[r].flags;
    sim->dist_epoch += 1 + (unsigned long long)ncycles * sim->n_stages;   // entry + one per stage and cycle
  }
  if (sim->flags & GEM_F_PROFILE) {
    const uint32_t pc = (uint32_t)std::min<uint64_t>(ncycles, 256);
    if (!sim->d_prof || sim->prof_cycles < pc) {
      if (sim->d_prof) cudaFree(sim->d_prof);
      sim->d_prof = nullptr;
      CK(dalloc(&sim->d_prof, (size_t)256 * sim->grid * GEM_PROF_SLOTS * 8));
    }
    sim->prof_cycles = pc;
    CK(cudaMemsetAsync(sim->d_prof, 0, (size_t)256 * sim->grid * GEM_PROF_SLOTS * 8, sim->stream));
    kp.prof = sim->d_prof;
    kp.prof_cycles = pc;
  }
  CK(cudaMemsetAsync(sim->d_bar, 0, (size_t)(GEM_BAR_MAX_CTAS + 2) * GEM_BAR_STRIDE * 8, sim->stream));
  if (sim->flags & GEM_F_DIGEST)
    CK(cudaMemsetAsync(sim->d_digest, 0, (size_t)sim->n_streams * sim->out_cap * 8, sim->stream));
  if (sim->lanes) {
    kp.lprog = sim->d_lprog;
    kp.pi_lane = sim->d_pi_lane;
    kp.po_lane = sim->d_po_lane;
    kp.n_groups = sim->n_groups;
    kp.ramp_words = sim->ramp_words;
    kp.state_words = sim->lane_words;
    kp.group = sim->lane_groups;
  }
  if (sim->words) {
    kp.lprog = sim->d_wprog;
    kp.state_words = sim->word_state;
    kp.loc_words = sim->local ? sim->loc_words : 0u;
  }
  void* args[] = {&kp};
  CK(cudaEventRecord(sim->ev0, sim->stream));
  CK(cudaLaunchCooperativeKernel(sim->words ? word_kernel_for(sim) : sim->lanes ? lane_kernel_for(sim->lane_groups, sim->lane_v2, sim->lane_m) : step_kernel_for(sim),
                                 dim3(sim->grid), dim3(sim->words ? GEM_WORD_THREADS : GEM_THREADS), args, sim->smem_bytes, sim->stream));
  CK(cudaEventRecord(sim->ev1, sim->stream));
  sim->in_head += (uint32_t)ncycles;
  sim->cycle += ncycles;
  sim->last_cycles = (uint32_t)ncycles;
  if (!(sim->flags & GEM_F_ASYNC)) {
    CK(cudaStreamSynchronize(sim->stream));
    CK(cudaEventElapsedTime(&sim->last_ms, sim->ev0, sim->ev1));
  }
  return GEM_OK;
}

int gem_bench_floor(int device, uint32_t grid, uint32_t iters, double* layer_clk, double* barrier_clk) {
  gem_sim* sim = nullptr;
  if (!layer_clk || !barrier_clk || !grid || grid > GEM_BAR_MAX_CTAS || !iters) return fail(GEM_E_INVAL, "bad floor request");
  CK(cudaSetDevice(device));
  unsigned long long *d_out = nullptr, *d_bar = nullptr;
  uint32_t* d_err = nullptr;
  CK(dalloc(&d_out, 64));
  CK(dalloc(&d_bar, (size_t)(GEM_BAR_MAX_CTAS + 2) * GEM_BAR_STRIDE * 8));
  CK(dalloc(&d_err, 64));
  CK(cudaMemset(d_bar, 0, (size_t)(GEM_BAR_MAX_CTAS + 2) * GEM_BAR_STRIDE * 8));
  unsigned long long h[2] = {0, 0};
  floor_layer_kernel<<<1, GEM_THREADS>>>(d_out, 64);
  floor_layer_kernel<<<1, GEM_THREADS>>>(d_out, iters);
  CK(cudaGetLastError());
  CK(cudaMemcpy(h, d_out, 16, cudaMemcpyDeviceToHost));
  *layer_clk = (double)h[0];
  KParams kp;
  memset(&kp, 0, sizeof(kp));
  kp.bar = d_bar;
  kp.err = d_err;
  void* args[] = {(void*)&kp, (void*)&d_out, (void*)&iters};
  CK(cudaLaunchCooperativeKernel((const void*)floor_barrier_kernel, dim3(grid), dim3(GEM_THREADS), args, 0, 0));
  CK(cudaMemcpy(h, d_out, 16, cudaMemcpyDeviceToHost));
  *barrier_clk = (double)h[0];
  cudaFree(d_out);
  cudaFree(d_bar);
  cudaFree(d_err);
  return GEM_OK;
}

int gem_bench_floor_step(int device, uint32_t iters, double* step_clk) {
  gem_sim* sim = nullptr;
  if (!step_clk || !iters) return fail(GEM_E_INVAL, "bad floor request");
  CK(cudaSetDevice(device));
  unsigned long long* d_out = nullptr;
  CK(dalloc(&d_out, 64));
  unsigned long long h = 0;
  floor_step_kernel<<<1, GEM_THREADS>>>(d_out, 64);
  floor_step_kernel<<<1, GEM_THREADS>>>(d_out, iters);
  CK(cudaGetLastError());
  CK(cudaMemcpy(&h, d_out, 8, cudaMemcpyDeviceToHost));
  cudaFree(d_out);
  *step_clk = (double)h;
  return GEM_OK;
}

int gem_last_step_ms(gem_sim* sim, float* ms) {
  if (int r = check(sim)) return r;
  if (!ms) return fail(GEM_E_INVAL, "null");
  CK(cudaEventSynchronize(sim->ev1));
  CK(cudaEventElapsedTime(&sim->last_ms, sim->ev0, sim->ev1));
  *ms = sim->last_ms;
  return GEM_OK;
}

int gem_read_outputs(gem_sim* sim, uint32_t* dst, uint64_t ncycles, int dst_on_device) {
  if (int r = check(sim)) return r;
  if (!dst || ncycles > sim->last_cycles) return fail(GEM_E_INVAL, "bad output request");
  if (!ncycles) return GEM_OK;
  CK(cudaSetDevice(sim->device));
  const size_t bytes = (size_t)sim->n_streams * ncycles * sim->po_words_ext * 4;
  uint32_t* out = dst;
  if (!dst_on_device) {
    if (int r = ensure_scratch(sim, bytes)) return r;
    out = sim->d_scratch;
  }
  if (sim->lanes) {
    const uint64_t warps = ncycles * sim->n_groups * sim->po_words_int;
    from_lanes_kernel<<<(unsigned)std::min<uint64_t>(65535, (warps * 32 + 255) / 256), 256, 0, sim->stream>>>(
        sim->d_po_lane, sim->d_po, sim->n_streams, (uint32_t)ncycles, sim->po_words_int,
        (uint64_t)sim->out_cap * sim->po_words_int, sim->po_words_int, sim->n_groups);
    CK(cudaGetLastError());
  }
  // rows = stream*ncycles + cycle; in-row stride = po_words_int, with stream stride out_cap
  // (one launch for all streams)
  {
    const uint64_t rows = (uint64_t)sim->n_streams * ncycles;
    unpermute_kernel<<<(unsigned)std::min<uint64_t>(4096, (rows * sim->po_words_ext + 255) / 256 + 1), 256, 0,
                       sim->stream>>>(sim->d_po, out, sim->d_po_int_of_ext, sim->n_po, sim->po_words_int,
                                      sim->po_words_ext, rows, sim->po_words_int, sim->po_words_ext, ncycles,
                                      (uint64_t)sim->out_cap * sim->po_words_int);
  }
  CK(cudaGetLastError());
  if (!dst_on_device) CK(cudaMemcpyAsync(dst, out, bytes, cudaMemcpyDeviceToHost, sim->stream));
  CK(cudaStreamSynchronize(sim->stream));
  return GEM_OK;
}

int gem_read_state(gem_sim* sim, uint32_t* dst, int dst_on_device) {
  if (int r = check(sim)) return r;
  if (!dst) return fail(GEM_E_INVAL, "null");
  CK(cudaSetDevice(sim->device));
  CK(cudaStreamSynchronize(sim->stream));
  const uint32_t buf = (uint32_t)(sim->cycle & 1);
  const size_t bytes = (size_t)sim->n_streams * sim->q_words_ext * 4;
  const size_t ibytes = (size_t)sim->n_streams * sim->q_words_int * 4;
  if (int r = ensure_scratch(sim, bytes + ibytes)) return r;
  uint32_t* out = dst_on_device ? dst : sim->d_scratch;
  const uint32_t* qin = sim->d_q + (size_t)buf * sim->n_streams * sim->q_words_int;
  if (sim->lanes) {
    uint32_t* tmp = sim->d_scratch + bytes / 4;
    const uint64_t warps = (uint64_t)sim->n_groups * sim->q_words_int;
    from_lanes_kernel<<<(unsigned)std::min<uint64_t>(65535, (warps * 32 + 255) / 256), 256, 0, sim->stream>>>(
        sim->d_q + (size_t)buf * sim->q_words_int * 32 * sim->n_groups, tmp, sim->n_streams, 1, sim->q_words_int,
        sim->q_words_int, 0, sim->n_groups);
    CK(cudaGetLastError());
    qin = tmp;
  }
  unpermute_kernel<<<std::min<uint64_t>(4096, ((uint64_t)sim->n_streams * sim->q_words_ext + 255) / 256 + 1), 256,
                     0, sim->stream>>>(qin, out,
                                       sim->d_q_int_of_ext, sim->n_flops, sim->q_words_int, sim->q_words_ext,
                                       sim->n_streams, sim->q_words_int, sim->q_words_ext);
  CK(cudaGetLastError());
  if (!dst_on_device) CK(cudaMemcpyAsync(dst, out, bytes, cudaMemcpyDeviceToHost, sim->stream));
  CK(cudaStreamSynchronize(sim->stream));
  return GEM_OK;
}

int gem_write_state(gem_sim* sim, const uint32_t* src, int src_on_device) {
  if (int r = check(sim)) return r;
  if (!src) return fail(GEM_E_INVAL, "null");
  CK(cudaSetDevice(sim->device));
  const uint32_t buf = (uint32_t)(sim->cycle & 1);
  const size_t bytes = (size_t)sim->n_streams * sim->q_words_ext * 4;
  if (int r = ensure_scratch(sim, bytes)) return r;
  CK(cudaMemcpyAsync(sim->d_scratch, src, bytes, src_on_device ? cudaMemcpyDeviceToDevice : cudaMemcpyHostToDevice,
                     sim->stream));
  uint32_t* qdst = sim->d_q + (size_t)buf * sim->n_streams * sim->q_words_int;
  if (sim->lanes) {
    if (int r = ensure_scratch(sim, bytes + (size_t)sim->n_streams * sim->q_words_int * 4)) return r;
    CK(cudaMemcpyAsync(sim->d_scratch, src, bytes, src_on_device ? cudaMemcpyDeviceToDevice : cudaMemcpyHostToDevice,
                       sim->stream));
    qdst = sim->d_scratch + bytes / 4;
  }
  permute_kernel<<<std::min<uint64_t>(4096, ((uint64_t)sim->n_streams * sim->q_words_int + 255) / 256 + 1), 256, 0,
                   sim->stream>>>(sim->d_scratch, qdst, sim->d_q_ext_of_int, sim->q_words_int, sim->q_words_ext,
                                  sim->n_streams);
  CK(cudaGetLastError());
  if (sim->lanes) {
    const uint64_t warps = (uint64_t)sim->n_groups * sim->q_words_int;
    to_lanes_kernel<<<(unsigned)std::min<uint64_t>(65535, (warps * 32 + 255) / 256), 256, 0, sim->stream>>>(
        qdst, sim->d_q + (size_t)buf * sim->q_words_int * 32 * sim->n_groups, sim->n_streams, 1, sim->q_words_int,
        sim->q_words_int, 0, sim->n_groups, 0);
    CK(cudaGetLastError());
  }
  CK(cudaStreamSynchronize(sim->stream));
  return GEM_OK;
}

int gem_read_state_trace(gem_sim* sim, uint32_t* dst, uint64_t ncycles) {
  if (int r = check(sim)) return r;
  if (!(sim->flags & GEM_F_TRACE_STATE)) return fail(GEM_E_INVAL, "GEM_F_TRACE_STATE not set");
  if (!dst || ncycles > sim->last_cycles) return fail(GEM_E_INVAL, "bad trace request");
  CK(cudaSetDevice(sim->device));
  CK(cudaStreamSynchronize(sim->stream));
  const size_t row = (size_t)ncycles * sim->q_words_ext * 4;
  CK(cudaMemcpy2D(dst, row, sim->d_qtrace, (size_t)sim->out_cap * sim->q_words_ext * 4, row, sim->n_streams,
                  cudaMemcpyDeviceToHost));
  return GEM_OK;
}

int gem_read_digests(gem_sim* sim, uint64_t* dst, uint64_t ncycles) {
  if (int r = check(sim)) return r;
  if (!(sim->flags & GEM_F_DIGEST)) return fail(GEM_E_INVAL, "GEM_F_DIGEST not set");
  if (!dst || ncycles > sim->last_cycles) return fail(GEM_E_INVAL, "bad digest request");
  CK(cudaSetDevice(sim->device));
  CK(cudaStreamSynchronize(sim->stream));
  const size_t row = (size_t)ncycles * 8;
  CK(cudaMemcpy2D(dst, row, sim->d_digest, (size_t)sim->out_cap * 8, row, sim->n_streams, cudaMemcpyDeviceToHost));
  return GEM_OK;
}

int gem_read_ram(gem_sim* sim, uint32_t ram_id, uint32_t stream, uint32_t* words) {
  if (int r = check(sim)) return r;
  if (!words || ram_id >= sim->n_rams || stream >= sim->n_streams) return fail(GEM_E_INVAL, "bad ram request");
  CK(cudaSetDevice(sim->device));
  CK(cudaStreamSynchronize(sim->stream));
  CK(cudaMemcpy(words, sim->d_mem + ((size_t)stream * sim->n_rams + ram_id) * GEM_RAM_WORDS, GEM_RAM_WORDS * 4,
                cudaMemcpyDeviceToHost));
  return GEM_OK;
}

int gem_write_ram(gem_sim* sim, uint32_t ram_id, uint32_t stream, const uint32_t* words) {
  if (int r = check(sim)) return r;
  if (!words || ram_id >= sim->n_rams || stream >= sim->n_streams) return fail(GEM_E_INVAL, "bad ram request");
  CK(cudaSetDevice(sim->device));
  CK(cudaStreamSynchronize(sim->stream));
  CK(cudaMemcpy(sim->d_mem + ((size_t)stream * sim->n_rams + ram_id) * GEM_RAM_WORDS, words, GEM_RAM_WORDS * 4,
                cudaMemcpyHostToDevice));
  return GEM_OK;
}

int gem_read_profile(gem_sim* sim, uint64_t* dst, uint32_t* n_cycles, uint32_t* grid) {
  if (int r = check(sim)) return r;
  if (!(sim->flags & GEM_F_PROFILE) || !sim->d_prof) return fail(GEM_E_INVAL, "GEM_F_PROFILE not set / no step yet");
  CK(cudaSetDevice(sim->device));
  CK(cudaStreamSynchronize(sim->stream));
  if (n_cycles) *n_cycles = sim->prof_cycles;
  if (grid) *grid = sim->grid;
  if (dst) CK(cudaMemcpy(dst, sim->d_prof, (size_t)sim->prof_cycles * sim->grid * GEM_PROF_SLOTS * 8, cudaMemcpyDeviceToHost));
  return GEM_OK;
}

int gem_read_activity(gem_sim* sim, uint64_t* evaluated, uint64_t* skipped) {
  if (int r = check(sim)) return r;
  if (!evaluated || !skipped) return fail(GEM_E_INVAL, "null argument");
  if (!(sim->flags & GEM_F_ACTIVITY)) return fail(GEM_E_INVAL, "GEM_F_ACTIVITY not set");
  CK(cudaSetDevice(sim->device));
  CK(cudaStreamSynchronize(sim->stream));
  unsigned long long h[2] = {0, 0};
  CK(cudaMemcpy(h, sim->d_act, 16, cudaMemcpyDeviceToHost));
  *evaluated = h[0];
  *skipped = h[1];
  return GEM_OK;
}

int gem_dist_owner(const void* blob, size_t nbytes, uint32_t world, uint32_t* owner) {
  if (!blob || !owner || world == 0 || world > GEM_DIST_MAX || nbytes < GH_N_WORDS * 4 || (nbytes & 3))
    return fail(GEM_E_INVAL, "bad arguments");
  const uint32_t* w = (const uint32_t*)blob;
  const size_t nw = nbytes / 4;
  if (w[GH_MAGIC] != GEM_MAGIC || w[GH_VERSION] != GEM_VERSION) return fail(GEM_E_FORMAT, "bad blob magic/version");
  const uint64_t total_words = w[GH_TOTAL_WORDS_LO] | ((uint64_t)w[GH_TOTAL_WORDS_HI] << 32);
  if (total_words != nw) return fail(GEM_E_FORMAT, "truncated blob");
  if (int r = validate_blob(w, nw)) return r;
  dist_assign(w + w[GH_OFF_PARTS], w + w[GH_OFF_STAGES], w[GH_N_STAGES], world, owner);
  return GEM_OK;
}

int gem_dist_export(gem_sim* sim, uint64_t max_cycles, gem_dist_buffers* out) {
  if (int r = check(sim)) return r;
  if (!out || sim->dist_world < 2) return fail(GEM_E_INVAL, "not a dist handle (gem_config::dist_world < 2)");
  if (max_cycles == 0 || max_cycles > 0xFFFFFFF0ull) return fail(GEM_E_INVAL, "bad max_cycles");
  CK(cudaSetDevice(sim->device));
  if (!sim->dist_exported) {
    if (int r = ensure_out(sim, (uint32_t)max_cycles)) return r;
    const size_t fb = (size_t)GEM_DIST_MAX * GEM_BAR_MAX_CTAS * GEM_BAR_STRIDE * 8;
    CK(dalloc(&sim->d_dist_flags, fb));
    CK(cudaMemset(sim->d_dist_flags, 0, fb));
    CK(cudaDeviceSynchronize());
    sim->dist_exported = true;
  } else if (max_cycles > sim->out_cap) {
    return fail(GEM_E_INVAL, "already exported with a smaller max_cycles");
  }
  out->q = sim->d_q; out->rd = sim->d_rd; out->cut = sim->d_cut; out->po = sim->d_po; out->flags = sim->d_dist_flags;
  out->grid = sim->grid;
  out->reserved = 0;
  return GEM_OK;
}

int gem_dist_ipc_handles(gem_sim* sim, void* out) {
  if (int r = check(sim)) return r;
  if (!out || !sim->dist_exported) return fail(GEM_E_INVAL, "gem_dist_export first");
  CK(cudaSetDevice(sim->device));
  cudaIpcMemHandle_t h[5];
  void* ptrs[5] = {sim->d_q, sim->d_rd, sim->d_cut, sim->d_po, sim->d_dist_flags};
  for (int k = 0; k < 5; k++) CK(cudaIpcGetMemHandle(&h[k], ptrs[k]));
  static_assert(sizeof(h) + 8 == GEM_DIST_IPC_BYTES, "IPC handle size");
  const uint32_t tail[2] = {sim->grid, 0u};
  std::memcpy(out, h, sizeof(h));
  std::memcpy((char*)out + sizeof(h), tail, 8);
  return GEM_OK;
}

int gem_dist_ipc_open(gem_sim* sim, const void* handles, gem_dist_buffers* out) {
  if (int r = check(sim)) return r;
  if (!handles || !out) return fail(GEM_E_INVAL, "null argument");
  CK(cudaSetDevice(sim->device));
  cudaIpcMemHandle_t h[5];
  std::memcpy(h, handles, sizeof(h));
  uint32_t tail[2];
  std::memcpy(tail, (const char*)handles + sizeof(h), 8);
  void* p[5] = {};
  for (int k = 0; k < 5; k++) {
    CK(cudaIpcOpenMemHandle(&p[k], h[k], cudaIpcMemLazyEnablePeerAccess));
    sim->ipc_opened.push_back(p[k]);
  }
  out->q = p[0]; out->rd = p[1]; out->cut = p[2]; out->po = p[3]; out->flags = p[4];
  out->grid = tail[0];
  out->reserved = 0;
  return GEM_OK;
}

int gem_dist_connect(gem_sim* sim, const gem_dist_buffers* peers) {
  if (int r = check(sim)) return r;
  if (!peers || !sim->dist_exported) return fail(GEM_E_INVAL, "gem_dist_export first");
  CK(cudaSetDevice(sim->device));
  for (uint32_t r = 0; r < sim->dist_world; r++) {
    if (r == sim->dist_rank) {   // this rank's own buffers
      sim->peers[r] = gem_dist_buffers{sim->d_q, sim->d_rd, sim->d_cut, sim->d_po, sim->d_dist_flags, sim->grid, 0};
      continue;
    }
    const gem_dist_buffers& b = peers[r];
    if (!b.q || !b.rd || !b.cut || !b.po || !b.flags) return fail(GEM_E_INVAL, "null peer buffer");
    if (b.grid == 0 || b.grid > GEM_BAR_MAX_CTAS) return fail(GEM_E_INVAL, "bad peer grid");
    cudaPointerAttributes a{};
    CK(cudaPointerGetAttributes(&a, b.q));
    if (a.type == cudaMemoryTypeDevice && a.device != sim->device) {   // same process, another device
      int can = 0;
      CK(cudaDeviceCanAccessPeer(&can, sim->device, a.device));
      if (!can) return fail(GEM_E_UNSUPPORTED, "no peer access between the devices");
      const cudaError_t e = cudaDeviceEnablePeerAccess(a.device, 0);
      if (e == cudaErrorPeerAccessAlreadyEnabled) (void)cudaGetLastError();
      else CK(e);
    }
    sim->peers[r] = b;
  }
  sim->dist_connected = true;
  return GEM_OK;
}

void gem_free(gem_sim* sim) {
  if (!sim) return;
  cudaSetDevice(sim->device);
  if (sim->stream) cudaStreamSynchronize(sim->stream);
  for (void* p : {(void*)sim->d_prog, (void*)sim->d_parts, (void*)sim->d_stage, (void*)sim->d_q_int_of_ext,
                  (void*)sim->d_q_ext_of_int, (void*)sim->d_po_int_of_ext, (void*)sim->d_q, (void*)sim->d_rd,
                  (void*)sim->d_cut, (void*)sim->d_mem, (void*)sim->d_pi, (void*)sim->d_po, (void*)sim->d_qtrace,
                  (void*)sim->d_scratch, (void*)sim->d_digest, (void*)sim->d_bar,
                  (void*)sim->d_prof, (void*)sim->d_wl_off, (void*)sim->d_wl_items, (void*)sim->d_lprog, (void*)sim->d_wprog,
                  (void*)sim->d_pi_lane, (void*)sim->d_po_lane, (void*)sim->d_act,
                  (void*)sim->d_dyn_units, (void*)sim->d_dyn_ctr, (void*)sim->d_dist_flags})
    if (p) cudaFree(p);
  for (void* p : sim->ipc_opened) cudaIpcCloseMemHandle(p);
  if (sim->ev0) cudaEventDestroy(sim->ev0);
  if (sim->ev1) cudaEventDestroy(sim->ev1);
  if (sim->ev_in) cudaEventDestroy(sim->ev_in);
  if (sim->h_err) cudaFreeHost(sim->h_err);
  if (sim->own_stream && sim->stream) cudaStreamDestroy(sim->stream);
  delete sim;
}

}  // extern "C"
